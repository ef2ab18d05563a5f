cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02c
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02c/build.log 2>&1; echo build rc $?
timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 2>&1 | tee gpurun_out/r02c/attn_v2.txt
TCB_ATTN=v1 timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 2>&1 | tee gpurun_out/r02c/attn_v1.txt
timeout 300 ncu --set full --clock-control none --import-source on -k regex:attn_tc2 -s 3 -c 1 -o gpurun_out/r02c/v2_c3 python scripts/attn_bench.py c3 > gpurun_out/r02c/ncu_v2.log 2>&1; echo ncu v2 rc $?
TCB_ATTN=v1 timeout 300 ncu --set full --clock-control none --import-source on -k regex:attn_tc_kernel -s 3 -c 1 -o gpurun_out/r02c/v1_c3 python scripts/attn_bench.py c3 > gpurun_out/r02c/ncu_v1.log 2>&1; echo ncu v1 rc $?
