cd $GRAFT_REPO_ROOT
python scripts/attn_bench.py c2 c3 c5 2>&1 | grep -v Warn
timeout 300 ncu --set full --clock-control none --import-source on -k regex:attn_bf16 -s 3 -c 1 -o gpurun_out/attn_c2 python scripts/attn_bench.py c2 > /dev/null 2>&1; echo ncu rc $?
