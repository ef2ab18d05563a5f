# HISTORICAL (r02): the TCB_LNG_UNIT=128 option this script A/Bs was measured slower and removed
# TCB_LNG_UNIT=128 vs 256: parity (op tests + forward parity) then per-class timing on c2
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-lngu}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
TCB_LNG_UNIT=128 timeout 600 python -m pytest -x -q tests/test_gpu_kernels.py -k "linear_ln" tests/test_gpu_parity.py > $T/pytest.log 2>&1; echo pytest rc $?; tail -3 $T/pytest.log
for r in 1 2; do for e in "TCB_LNG_UNIT=256" "TCB_LNG_UNIT=128"; do
  echo "== env[$e] round $r"; env $e timeout 300 python scripts/r02/bench_classes.py c2 2>&1 | grep -v '"us": 0' | tee -a $T/out.txt
done; done
for e in "TCB_LN_KERNEL=global TCB_LNG_UNIT=128" "TCB_LN_KERNEL=global TCB_LNG_UNIT=256"; do
  echo "== env[$e]"; env $e timeout 300 python scripts/r02/bench_classes.py c2 2>&1 | grep -v '"us": 0' | tee -a $T/out.txt
done
