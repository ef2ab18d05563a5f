# A/B two variants of one source file in ONE run (same box, same clocks):
#   ALT=<path of the B version>  DST=<repo-relative file it replaces>  WL="c2 c3 ..."  TAG=...
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-ab}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/buildA.log 2>&1; echo buildA rc $?
[ -n "$TESTK" ] && { timeout 600 python -m pytest tests -m gpu -q -x -k "$TESTK" -p no:cacheprovider --timeout 120 > $T/pytest.log 2>&1; echo pytest rc $?; tail -2 $T/pytest.log; }
rm -rf /tmp/repoB; mkdir -p /tmp/repoB; cp -r . /tmp/repoB/ 2>/dev/null; cp $ALT /tmp/repoB/$DST
(cd /tmp/repoB && python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1; echo buildB rc $?)
for r in 1 2; do
  echo "== A (current) round $r"; timeout 300 python ${BENCH:-scripts/attn_bench.py} ${WL:-c2 c3 c4 c5} 2>&1 | tee -a $T/A.txt
  echo "== B ($ALT) round $r"; (cd /tmp/repoB && timeout 300 python ${BENCH:-scripts/attn_bench.py} ${WL:-c2 c3 c4 c5} 2>&1) | tee -a $T/B.txt
done
