# r02 evidence: bench lines (C2-C5), ncu launch list of one eager C2 step, one ncu --set full
# capture per kernel class (C2 + the d = 768 / 1024 LN kernels), GPU tests.  -> gpurun_out/$TAG
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-r02prof}; mkdir -p $T/full
export NCU_ENV="TCB_NO_COOP=1"
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1 || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
if [ -z "$SKIP_TESTS" ]; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $T/smoke.log 2>&1; echo smoke rc $?; tail -1 $T/smoke.log
  timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 --timeout_method thread > $T/pytest_gpu.log 2>&1; echo pytest rc $?; tail -2 $T/pytest_gpu.log
fi
for w in ${WORKLOADS-c2 c3 c4 c5}; do
  timeout 600 python bench.py --steps 20 --warmup 5 --workload $w > $T/bench_$w.json 2> $T/bench_$w.err; echo bench $w rc $?
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $T/launches.csv env $NCU_ENV python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-graph > $T/ncu_launch.log 2>&1; echo launches rc $?
i=0
while read -r w k; do
  [ -z "$w" ] && continue
  i=$((i+1))
  timeout 600 ncu --set full --clock-control none --import-source on \
    -k "regex:$k" -s 6 -c 1 -o $T/full/${w}_$(echo "$k" | tr -c "a-zA-Z0-9\n" "_") env $NCU_ENV python bench.py --workload $w --steps 1 --warmup 2 --no-cpu-baseline --no-graph > $T/ncu_full_$i.log 2>&1; echo full $i $w $k rc $?
done <<LIST
${LIST:-c2 linear_tc_kernel<2, 256, 0>
c2 attn_tc3s_kernel
c2 linear_ln_kernel
c2 linear_tc_kernel<2, 256, 2>
c2 linear_lng_kernel<2>
c2 pack_embed
c2 unpack_kernel
c3 attn_tc3_kernel
c3 linear_lnc_kernel<3>
c3 linear_lng_kernel<3>
c4 linear_lnc_kernel<4>
c4 linear_lng_kernel<4>}
LIST
