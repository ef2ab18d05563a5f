cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-xov}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $T/smoke.log 2>&1; echo smoke rc $?; tail -2 $T/smoke.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 240 --timeout_method thread > $T/pytest_parity.log 2>&1; echo parity rc $?; tail -3 $T/pytest_parity.log
IFS='|' read -ra SETS <<< "${ENVS:-TCB_NO_XOVERLAP=1|X=1}"
for r in 1 2; do for e in "${SETS[@]}"; do
  echo "== env[$e] round $r"; env $e timeout 300 python scripts/r02/bench_classes.py ${WL:-c2 c3} 2>&1 | tee -a $T/out.txt
done; done
