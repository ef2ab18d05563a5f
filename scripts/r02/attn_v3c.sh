# attention v3: parity + op benchmark + probe build (tag in $TAG)
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-r02x}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or attn" -p no:cacheprovider > $T/pytest_attn.log 2>&1; echo pytest attn rc $?; tail -3 $T/pytest_attn.log
timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 2>&1 | tee $T/attn.txt
if [ -n "$PROBE" ]; then
  cp paper_conf_icpp_fuc0z22_b200/_build.py /tmp/_b.py
  sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_ATTN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
  python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > $T/build_probe.log 2>&1
  for w in c2 c3; do timeout 120 python scripts/attn_bench.py $w 2>&1 | grep -E "a3probe|workload" | tail -7; done | tee $T/probe.txt
  cp /tmp/_b.py paper_conf_icpp_fuc0z22_b200/_build.py
fi
