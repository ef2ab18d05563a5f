cd $GRAFT_REPO_ROOT
ALT=scripts/r02/alt_attn_pre_epi.cu DST=paper_conf_icpp_fuc0z22_b200/csrc/attention_tc.cu TESTK="attention" BENCH=scripts/r02/bench_classes.py WL="c2" TAG=attn_v3s_epi bash scripts/r02/ab_two.sh
LIST='c3 gemm_ffn1 6 linear_tc_kernel<.int.2, .int.256, .int.1>
c4 gemm_ffn1 6 linear_tc_kernel<.int.2, .int.256, .int.1>
c2 attention 6 attn_tc3s_kernel' TAG=r02full3 NOBUILD=1 bash scripts/r02/profile_full.sh
