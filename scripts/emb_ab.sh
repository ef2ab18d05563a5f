cd $GRAFT_REPO_ROOT
for c in 64 16 8; do
  TCB_EXTRA_NVCC_FLAGS="-DTCB_ROW_CHUNK=$c" python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build()" > /dev/null 2>&1
  echo "chunk $c"; python scripts/ops_bench.py 2>&1 | grep -i -E "embed|unpack" | head -8
done
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -m gpu -q -x --timeout 300 --timeout_method thread -p no:cacheprovider 2>&1 | tail -2
