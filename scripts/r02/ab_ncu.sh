cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-abncu}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/buildA.log 2>&1; echo buildA rc $?
rm -rf /tmp/repoB; mkdir -p /tmp/repoB; cp -r . /tmp/repoB/ 2>/dev/null; cp $ALT /tmp/repoB/$DST
(cd /tmp/repoB && python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1; echo buildB rc $?)
timeout 300 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-attn_tc3} -s 3 -c 1 -o $T/A python scripts/attn_bench.py ${WL:-c3} > $T/ncuA.log 2>&1; echo ncuA rc $?
(cd /tmp/repoB && timeout 300 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-attn_tc3} -s 3 -c 1 -o $GRAFT_REPO_ROOT/$T/B python scripts/attn_bench.py ${WL:-c3} > $GRAFT_REPO_ROOT/$T/ncuB.log 2>&1; echo ncuB rc $?)
