# Evidence for profiles/: bench lines (C2-C5), ncu launch list of one eager C2 step, one
# ncu --set full capture per kernel class of C2 (+ the C4 LN-fused GEMMs).  Run via gpurun.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/prof
# ncu replays kernels one at a time and rejects cooperative cluster launches: plain launches
# for the captures (a single stream, so the L2-exchange kernel is co-resident anyway)
export NCU_ENV="TCB_NO_COOP=1"
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/prof/build.log 2>&1 || exit 1
for w in ${WORKLOADS-c2 c3 c4 c5}; do
  timeout 600 python bench.py --steps 20 --warmup 5 --workload $w > gpurun_out/prof/bench_$w.json 2> gpurun_out/prof/bench_$w.err; echo bench $w rc $?
done
[ -n "$SKIP_LAUNCHES" ] || timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/prof/launches.csv env $NCU_ENV python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-graph > gpurun_out/prof/ncu_launch.log 2>&1; echo launches rc $?
i=0
while read -r w k; do
  i=$((i+1))
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 6 -c 1 -o gpurun_out/prof/full_${w}_$(echo "$k" | tr -c "a-zA-Z0-9\n" "_") env $NCU_ENV python bench.py --workload $w --steps 1 --warmup 2 --no-cpu-baseline --no-graph > gpurun_out/prof/ncu_full_$i.log 2>&1; echo full $i $w $k rc $?
done <<LIST
${LIST:-c2 linear_tc_kernel.*256, .int.0
c2 attn_tc_kernel
c2 linear_ln_kernel<.bool.0>
c2 linear_tc_kernel.*256, .int.2
c2 linear_lng_kernel<.int.2>
c2 pack_embed
c2 unpack_kernel
c4 linear_lnc_kernel<.int.4>
c4 linear_lng_kernel<.int.4>}
LIST
