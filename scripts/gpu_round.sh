# Full GPU round-trip: smoke, GPU tests, bench on every workload.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo build rc $?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc $?
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 --timeout_method thread -p no:cacheprovider ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?
tail -15 gpurun_out/pytest_gpu.log
for w in ${WORKLOADS:-c2 c3 c4 c5}; do
  timeout 600 python bench.py --steps 20 --warmup 5 --workload $w > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; echo bench $w rc $?
  tail -2 gpurun_out/bench_$w.err
done
