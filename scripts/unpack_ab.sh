# unpack kernel: graph-timed op microbenchmark, then the GPU tests and bench lines.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo build rc $?
python scripts/ops_bench.py c2 c3 c4 c5 2>&1 | grep unpack
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 --timeout_method thread -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_gpu.log
for w in ${WORKLOADS:-c2 c3 c4 c5}; do
  timeout 600 python bench.py --steps 20 --warmup 5 --workload $w > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; echo bench $w rc $?
done
