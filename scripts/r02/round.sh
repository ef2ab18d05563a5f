# build, smoke, GPU tests, bench lines (C2-C5) -> gpurun_out/$TAG
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-r02}; mkdir -p $T
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $T/smoke.log 2>&1; echo smoke rc $?; tail -1 $T/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider ${PYTEST_K:+-k "$PYTEST_K"} > $T/pytest_gpu.log 2>&1; echo pytest rc $?; tail -4 $T/pytest_gpu.log
for w in ${WORKLOADS:-c2 c3 c4 c5}; do
  timeout 600 python bench.py --steps 20 --warmup 5 --workload $w ${BENCH_ARGS} > $T/bench_$w.json 2> $T/bench_$w.err; echo bench $w rc $?; tail -1 $T/bench_$w.err
done
