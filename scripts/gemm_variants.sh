cd $GRAFT_REPO_ROOT
for v in default cg1_256 cg2_128 cg1_128; do
  TCB_GEMM_VARIANT=$v timeout 300 python scripts/gemm_bench.py 2>&1 | grep -v Warning
done
