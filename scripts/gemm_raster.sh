cd $GRAFT_REPO_ROOT
for r in 0 4 8 16 32; do
  TCB_GEMM_RASTER=$r TCB_GEMM_VARIANT=r$r timeout 300 python scripts/gemm_bench.py 2>&1 | grep -v Warning
done
