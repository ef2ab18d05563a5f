cd $GRAFT_REPO_ROOT
ALT=scripts/r02/alt_attn_pre_defer.cu DST=paper_conf_icpp_fuc0z22_b200/csrc/attention_tc.cu TESTK="attention or parity" BENCH=scripts/r02/bench_classes.py WL="c2" TAG=attn_defer bash scripts/r02/ab_two.sh 2>&1 | grep -E "rc|passed|failed|==|attention|step"
