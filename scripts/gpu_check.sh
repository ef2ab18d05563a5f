# GPU round-trip: smoke, GPU tests, bench, ncu launch list + one full capture per hot kernel.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc $?
timeout 900 python -m pytest tests -m gpu -q --timeout 180 --timeout_method thread -p no:cacheprovider ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?
tail -15 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc $?
tail -3 gpurun_out/bench.err
if [ -n "$NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-graph > gpurun_out/ncu_bench.log 2>&1; echo ncu-launches rc $?
  for k in linear_tc attn_bf16 layernorm pack_embed; do
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 8 -c 2 \
      -o gpurun_out/full_$k python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-graph > gpurun_out/ncu_full_$k.log 2>&1; echo ncu-full $k rc $?
  done
fi
