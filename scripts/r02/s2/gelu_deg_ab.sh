# degree-4 GELU fit (default) vs degree 5 (-DTCB_GELU_DEG5): GEMM op tests, in-step FFN1 (C3, C4)
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-stream}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/buildA.log 2>&1; echo buildA rc $?
rm -rf /tmp/repoB; mkdir -p /tmp/repoB; cp -r . /tmp/repoB/ 2>/dev/null
(cd /tmp/repoB && TCB_EXTRA_NVCC_FLAGS=-DTCB_GELU_DEG5 python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1; echo buildB rc $?)
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "linear_bf16" -p no:cacheprovider --timeout 120 > $T/pytest_lin.log 2>&1; echo pytest lin rc $?; tail -2 $T/pytest_lin.log
for r in 1 2; do
  echo "== classes A round $r"; timeout 300 python scripts/r02/bench_classes.py c3 c4 2>&1 | grep 'step\|ffn1' | tee -a $T/classesA.txt
  echo "== classes B round $r"; (cd /tmp/repoB && timeout 300 python scripts/r02/bench_classes.py c3 c4 2>&1) | grep 'step\|ffn1' | tee -a $T/classesB.txt
done
