# S loads skipped for dead 32-key groups (default) vs loading every group (-DTCB_ATTN_LOAD_DEAD): attention
# tests, op benchmark and in-step classes, same box
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-stream}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/buildA.log 2>&1; echo buildA rc $?
rm -rf /tmp/repoB; mkdir -p /tmp/repoB; cp -r . /tmp/repoB/ 2>/dev/null
(cd /tmp/repoB && TCB_EXTRA_NVCC_FLAGS=-DTCB_ATTN_LOAD_DEAD python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1; echo buildB rc $?)
timeout 60 python scripts/attn_bench.py c2 c3 > $T/quick.txt 2>&1; echo quick rc $?; cat $T/quick.txt
grep -q '"us"' $T/quick.txt || exit 3
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" -p no:cacheprovider --timeout 120 > $T/pytest_attn.log 2>&1; echo pytest attn rc $?; tail -3 $T/pytest_attn.log
for r in 1 2; do
  echo "== A skip-dead round $r"; timeout 60 python scripts/attn_bench.py c2 c3 c4 c5 2>&1 | tee -a $T/opA.txt
  echo "== B load-all round $r"; (cd /tmp/repoB && timeout 60 python scripts/attn_bench.py c2 c3 c4 c5 2>&1) | tee -a $T/opB.txt
done
echo "== classes A"; timeout 300 python scripts/r02/bench_classes.py c2 c3 c4 c5 2>&1 | grep 'step\|attention' | tee -a $T/classesA.txt
echo "== classes B"; (cd /tmp/repoB && timeout 300 python scripts/r02/bench_classes.py c2 c3 c4 c5 2>&1) | grep 'step\|attention' | tee -a $T/classesB.txt
