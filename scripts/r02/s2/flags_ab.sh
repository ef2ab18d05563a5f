# the same source built with different extra nvcc flags (FLAGS_B, FLAGS_C), in-step classes on one box
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-flags}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/buildA.log 2>&1; echo buildA rc $?
for v in B C; do
  eval fl=\$FLAGS_$v; [ -z "$fl" ] && continue
  rm -rf /tmp/repo$v; mkdir -p /tmp/repo$v; cp -r . /tmp/repo$v/ 2>/dev/null
  (cd /tmp/repo$v && TCB_EXTRA_NVCC_FLAGS="$fl" python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1; echo build$v rc $?)
done
timeout 120 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention and not scheduler" -p no:cacheprovider --timeout 60 > $T/pytest.log 2>&1; echo pytestA rc $?
[ -n "$FLAGS_B" ] && (cd /tmp/repoB && timeout 120 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention and not scheduler" -p no:cacheprovider --timeout 60 > /dev/null 2>&1; echo pytestB rc $?)
for r in 1 2; do
  echo "== A round $r"; timeout 300 python scripts/r02/bench_classes.py ${WL:-c2 c3} 2>&1 | grep -v 'embed\|unpack' | tee -a $T/A.txt
  for v in B C; do
    eval fl=\$FLAGS_$v; [ -z "$fl" ] && continue
    echo "== $v [$fl] round $r"; (cd /tmp/repo$v && timeout 300 python scripts/r02/bench_classes.py ${WL:-c2 c3} 2>&1) | grep -v 'embed\|unpack' | tee -a $T/$v.txt
  done
done
