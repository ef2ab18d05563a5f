cd $GRAFT_REPO_ROOT
ALT=scripts/r02/alt_api_e2e_old.cu DST=paper_conf_icpp_fuc0z22_b200/csrc/api.cu TESTK="session or parity or smoke" BENCH=scripts/r02/e2e_only.py WL="c2 c5" TAG=e2e bash scripts/r02/ab_two.sh
