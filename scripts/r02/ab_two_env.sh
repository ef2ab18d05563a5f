cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-ab}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/buildA.log 2>&1; echo buildA rc $?
rm -rf /tmp/repoB; mkdir -p /tmp/repoB; cp -r . /tmp/repoB/ 2>/dev/null; cp $ALT /tmp/repoB/$DST
(cd /tmp/repoB && python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1; echo buildB rc $?)
for e in "" "TCB_ATTN_STATIC=1"; do
  echo "== A env[$e]"; env $e timeout 300 python scripts/attn_bench.py ${WL:-c2 c3 c4 c5} 2>&1
  echo "== B env[$e]"; (cd /tmp/repoB && env $e timeout 300 python scripts/attn_bench.py ${WL:-c2 c3 c4 c5} 2>&1)
done
