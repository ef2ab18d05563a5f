# run $BENCH under several environment settings (ENVS="A=1 B=2|C=3|..."), one box
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-sweep}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
IFS='|' read -ra SETS <<< "$ENVS"
for r in 1 2; do for e in "${SETS[@]}"; do
  echo "== env[$e] round $r"; env $e timeout 300 python ${BENCH:-scripts/r02/bench_classes.py} ${WL:-c2} 2>&1 | tee -a $T/out.txt
done; done
