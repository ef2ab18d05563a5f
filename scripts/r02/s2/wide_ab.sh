# wide 256 x 512 A-resident tiles (K <= 512) vs the 256 x 256 tiles (TCB_GEMM_WIDE=0)
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-wide}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider --timeout 60 -k "linear" > $T/pytest_ops.log 2>&1; echo pytest ops rc $?; tail -2 $T/pytest_ops.log
timeout 400 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 200 -k "c2_transformer or unpacked or deterministic or c1_toy" > $T/pytest_parity.log 2>&1; echo pytest parity rc $?; tail -2 $T/pytest_parity.log
for r in 1 2; do
  for e in "TCB_GEMM_WIDE=0" "TCB_GEMM_WIDE=1"; do
    echo "== env[$e] round $r"; env $e timeout 300 python scripts/r02/bench_classes.py c2 c5 2>&1 | grep 'step\|qkv\|ffn1' | tee -a $T/classes.txt
  done
done
