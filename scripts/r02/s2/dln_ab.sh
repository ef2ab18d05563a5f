# deferred LN1 (default) vs TCB_LN1=fused: parity vs the oracle, then in-step per-class times
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-dln}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $T/smoke.log 2>&1; echo smoke rc $?; tail -2 $T/smoke.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 300 ${PYTEST_K:+-k "$PYTEST_K"} > $T/pytest_parity.log 2>&1; echo pytest parity rc $?; tail -3 $T/pytest_parity.log
for e in "TCB_X=0" "TCB_LN1=fused"; do
  echo "== classes env[$e]"; env $e timeout 300 python scripts/r02/bench_classes.py ${WLB:-c2 c3 c4 c5} 2>&1 | grep -v 'embed\|unpack' | tee -a $T/classes.txt
done
