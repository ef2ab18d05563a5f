cd $GRAFT_REPO_ROOT
ALT=scripts/r02/alt_attn_epi_only.cu DST=paper_conf_icpp_fuc0z22_b200/csrc/attention_tc.cu TESTK="attention or parity" TAG=attn_epi2 bash scripts/r02/ab_two.sh
echo "=== pre-epi reference"
(cd /tmp/repoB && cp $GRAFT_REPO_ROOT/scripts/r02/alt_attn_pre_epi.cu paper_conf_icpp_fuc0z22_b200/csrc/attention_tc.cu && python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1 && timeout 300 python scripts/attn_bench.py c2 c3 c4 c5)
