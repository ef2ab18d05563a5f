cd $GRAFT_REPO_ROOT
TAG=lngu bash scripts/r02/lng_unit.sh
TAG=r02full NOBUILD=1 KEEP="c2_gemm_ffn2 c3_attention" bash scripts/r02/profile_full.sh
