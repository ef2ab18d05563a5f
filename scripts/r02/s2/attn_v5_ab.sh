# v5 (separate epilogue warpgroup) vs v3 (TCB_ATTN=v3): attention tests, op bench, in-step classes
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-v5ab}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 60 python scripts/attn_bench.py c2 > $T/quick.txt 2>&1; echo quick rc $?; cat $T/quick.txt
grep -q '"us"' $T/quick.txt || exit 3
timeout 400 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" -p no:cacheprovider --timeout 60 > $T/pytest_attn.log 2>&1; echo pytest attn rc $?; tail -3 $T/pytest_attn.log
for r in 1 2; do
  for e in "TCB_X=0" "TCB_ATTN=v3"; do
    echo "== op env[$e] round $r"; env $e timeout 60 python scripts/attn_bench.py ${WL:-c2 c3 c4 c5} 2>&1 | tee -a $T/op.txt
  done
done
for e in "TCB_X=0" "TCB_ATTN=v3"; do
  echo "== classes env[$e]"; env $e timeout 200 python scripts/r02/bench_classes.py ${WLB:-c2 c3} 2>&1 | grep -v 'embed\|unpack' | tee -a $T/classes.txt
done
