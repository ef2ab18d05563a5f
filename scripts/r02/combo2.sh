cd $GRAFT_REPO_ROOT
TAG=emb bash scripts/r02/emb_ab.sh
LIST='c2 gemm_qkv 6 linear_tc_kernel<.int.2, .int.256, .int.0>
c2 gemm_ffn1 6 linear_tc_kernel<.int.2, .int.256, .int.2>
c2 gemm_ffn2 6 linear_lng_kernel<.int.2, .int.256>
c3 gemm_qkv 6 linear_tc_kernel<.int.2, .int.256, .int.0>
c3 gemm_o 6 linear_lnc_kernel<.int.3>
c3 gemm_ffn1 6 linear_tc_kernel<.int.2, .int.256, .int.2>
c3 gemm_ffn2 6 linear_lng_kernel<.int.3, .int.256>
c4 gemm_qkv 6 linear_tc_kernel<.int.2, .int.256, .int.0>
c4 gemm_o 6 linear_lnc_kernel<.int.4>
c4 gemm_ffn1 6 linear_tc_kernel<.int.2, .int.256, .int.2>
c4 gemm_ffn2 6 linear_lng_kernel<.int.4, .int.256>
c5 gemm_ffn2 6 linear_lng_kernel<.int.4, .int.256>
c5 gemm_ffn1 6 linear_tc_kernel<.int.2, .int.256, .int.2>
c5 embed 2 pack_embed
c4 embed 2 pack_embed
c3 embed 2 pack_embed
c2 embed 2 pack_embed' TAG=r02full2 NOBUILD=1 KEEP="c2_gemm_ffn2 c2_embed" bash scripts/r02/profile_full.sh
