cd $GRAFT_REPO_ROOT
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_ATTN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null
for w in c2 c4; do echo "W $w"; python scripts/attn_bench.py $w 2>&1 | grep -E "attnprobe|tcprobe|workload" | tail -6; done
