cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02d
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_ATTN2_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > gpurun_out/r02d/build.log 2>&1
for w in c2 c3; do timeout 120 python scripts/attn_bench.py $w 2>&1 | grep -E "a2probe|workload" | tail -7; done | tee gpurun_out/r02d/probe.txt
