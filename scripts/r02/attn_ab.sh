# attention v2 vs v1: parity tests + op benchmark + a C2/C3 bench line
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02b
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02b/build.log 2>&1; echo build rc $?
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or attn" -p no:cacheprovider > gpurun_out/r02b/pytest_attn.log 2>&1; echo pytest attn rc $?; tail -5 gpurun_out/r02b/pytest_attn.log
timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 > gpurun_out/r02b/attn_v2.txt 2>&1; echo v2 rc $?
TCB_ATTN=v1 timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 > gpurun_out/r02b/attn_v1.txt 2>&1; echo v1 rc $?
cat gpurun_out/r02b/attn_v2.txt gpurun_out/r02b/attn_v1.txt
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02b/pytest_gpu.log 2>&1; echo pytest gpu rc $?; tail -5 gpurun_out/r02b/pytest_gpu.log
for w in c2 c3; do timeout 300 python bench.py --steps 20 --warmup 5 --workload $w --no-cpu-baseline > gpurun_out/r02b/bench_$w.json 2>gpurun_out/r02b/bench_$w.err; echo bench $w rc $?; done
