cd $GRAFT_REPO_ROOT; T=gpurun_out/combo3; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 900 python -m pytest tests -m gpu -q -k "embed or unpack or parity" -p no:cacheprovider > $T/pytest.log 2>&1; echo pytest rc $?; tail -2 $T/pytest.log
timeout 600 python scripts/gemm_bench.py 2>&1 | tee $T/gemm_vs_cublas.jsonl
rm -rf /tmp/repoP; mkdir -p /tmp/repoP; cp -r . /tmp/repoP/ 2>/dev/null
cd /tmp/repoP && sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_ATTN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py && \
  python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1
for w in c3 c2; do echo "W $w"; timeout 300 python scripts/attn_bench.py $w 2>&1 | grep -E "probe|workload" | tail -8; done | tee $GRAFT_REPO_ROOT/$T/attn_probe.txt
