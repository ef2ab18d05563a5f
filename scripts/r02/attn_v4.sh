cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02h
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02h/build.log 2>&1; echo build rc $?
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or attn" -p no:cacheprovider > gpurun_out/r02h/pytest_attn.log 2>&1; echo pytest attn rc $?; tail -3 gpurun_out/r02h/pytest_attn.log
timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 2>&1 | tee gpurun_out/r02h/attn_v4.txt
timeout 300 ncu --set full --clock-control none --import-source on -k regex:attn_tc4 -s 3 -c 1 -o gpurun_out/r02h/v4_c3 python scripts/attn_bench.py c3 > gpurun_out/r02h/ncu_v4.log 2>&1; echo ncu v4 rc $?
