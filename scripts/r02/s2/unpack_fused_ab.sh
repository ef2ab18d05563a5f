# fused unpack (tcb_encoder_forward_unpacked) vs separate unpack: parity + session tests, then
# the bench step time per workload (TCB_BENCH_UNPACK=separate for B), same box
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-unpackfused}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 300 -k "unpacked or session or c2_transformer or full_bench or deterministic" > $T/pytest.log 2>&1; echo pytest rc $?; tail -3 $T/pytest.log
for r in 1 2; do
  for e in "TCB_X=0" "TCB_BENCH_UNPACK=separate"; do
    echo "== env[$e] round $r"; env $e timeout 300 python scripts/r02/bench_classes.py ${WL:-c2 c3 c5} 2>&1 | grep 'step\|ffn2\|unpack' | tee -a $T/classes.txt
  done
done
