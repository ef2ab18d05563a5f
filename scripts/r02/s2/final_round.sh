# end-of-round evidence with the final code: build, smoke, pytest -m gpu, bench lines C2-C5,
# ncu launch list of an eager C2 step, ncu --set full raw pages (CSV) per C2 class + C3
# attention / LN GEMMs -> gpurun_out/$TAG
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-final3}; mkdir -p $T/full /tmp/reps
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1 || exit 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $T/smoke.log 2>&1; echo smoke rc $?; tail -1 $T/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -rs -p no:cacheprovider --timeout 600 --timeout_method thread > $T/pytest_gpu.log 2>&1; echo pytest rc $?; tail -3 $T/pytest_gpu.log
for w in c2 c3 c4 c5; do
  timeout 600 python bench.py --steps 20 --warmup 5 --workload $w > $T/bench_$w.json 2> $T/bench_$w.err; echo bench $w rc $?
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $T/launches.csv env TCB_NO_COOP=1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-graph > $T/ncu_launch.log 2>&1; echo launches rc $?
while read -r w c s k; do
  [ -z "$w" ] && continue
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s $s -c 1 -f -o /tmp/reps/${w}_$c env TCB_NO_COOP=1 python bench.py --workload $w --steps 1 --warmup 2 \
    --no-cpu-baseline --no-graph > $T/full/${w}_$c.log 2>&1
  echo "full $w $c rc $?"
  ncu -i /tmp/reps/${w}_$c.ncu-rep --page raw --csv > $T/full/${w}_$c.csv 2>&1
done <<LIST
c2 gemm_qkv 6 linear_tc_kernel<2, 256, 0>
c2 gemm_o 6 linear_ln_kernel
c2 gemm_ffn1 6 linear_tc_kernel<2, 256, 2>
c2 gemm_ffn2 6 linear_lng_kernel<2
c2 attention 6 attn_tc3s_kernel
c2 embed 2 pack_embed
c3 gemm_o 6 linear_lnc_kernel<3>
c3 gemm_ffn2 6 linear_lng_kernel<3
c3 attention 6 attn_tc3_kernel
LIST
ls -la $T/full | head -30
