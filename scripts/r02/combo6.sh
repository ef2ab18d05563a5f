cd $GRAFT_REPO_ROOT
ALT=scripts/r02/alt_attn_pre_epi.cu DST=paper_conf_icpp_fuc0z22_b200/csrc/attention_tc.cu TESTK="attention or parity" TAG=attn_reorder bash scripts/r02/ab_two.sh
