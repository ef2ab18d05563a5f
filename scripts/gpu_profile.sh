# ncu evidence for profiles/: launch list of one eager bench step + one full capture per hot kernel
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
if [ -z "$SKIP_LAUNCHES" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-graph > gpurun_out/ncu_bench.log 2>&1; echo ncu-launches rc $?
fi
i=0
for k in ${KERNELS:-"linear_tc_kernel.*int.2, .int.256, .int.0" "linear_tc_kernel.*int.2, .int.256, .int.3" "linear_tc_kernel.*int.2, .int.256, .int.2" attn_bf16 layernorm pack_embed unpack}; do
  i=$((i+1))
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 6 -c 1 \
    -o gpurun_out/full_$i python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-graph > gpurun_out/ncu_full_$i.log 2>&1; echo ncu-full $i $k rc $?
done
