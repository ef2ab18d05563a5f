# one ncu --set full capture per (workload, kernel class); raw CSV kept, .ncu-rep dropped
# (the pull-back is capped) -> gpurun_out/$TAG/full/<wl>_<class>.csv
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-r02full}; mkdir -p $T/full /tmp/reps
[ -n "$NOBUILD" ] || python -c "import __graft_entry__ as g; g.build()" > $T/build_full.log 2>&1 || exit 1
while read -r w c s k; do
  [ -z "$w" ] && continue
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s $s -c 1 -f -o /tmp/reps/${w}_$c env TCB_NO_COOP=1 python bench.py --workload $w --steps 1 --warmup 2 \
    --no-cpu-baseline --no-graph > $T/full/${w}_$c.log 2>&1
  echo "full $w $c rc $?"
  ncu -i /tmp/reps/${w}_$c.ncu-rep --page raw --csv > $T/full/${w}_$c.csv 2>&1
  [ -n "$KEEP" ] && case " $KEEP " in *" ${w}_$c "*) cp /tmp/reps/${w}_$c.ncu-rep $T/full/ ;; esac
done <<LIST
${LIST:-c2 gemm_qkv 6 linear_tc_kernel<2, 256, 0>
c2 gemm_o 6 linear_ln_kernel
c2 gemm_ffn1 6 linear_tc_kernel<2, 256, 2>
c2 gemm_ffn2 6 linear_lng_kernel<2, 256>
c2 attention 6 attn_tc3s_kernel
c2 embed 2 pack_embed
c2 unpack 2 unpack_kernel
c3 gemm_qkv 6 linear_tc_kernel<2, 256, 0>
c3 gemm_o 6 linear_lnc_kernel<3>
c3 gemm_ffn1 6 linear_tc_kernel<2, 256, 2>
c3 gemm_ffn2 6 linear_lng_kernel<3, 256>
c3 attention 6 attn_tc3_kernel
c3 embed 2 pack_embed
c3 unpack 2 unpack_kernel
c4 gemm_qkv 6 linear_tc_kernel<2, 256, 0>
c4 gemm_o 6 linear_lnc_kernel<4>
c4 gemm_ffn1 6 linear_tc_kernel<2, 256, 2>
c4 gemm_ffn2 6 linear_lng_kernel<4, 256>
c4 attention 6 attn_tc3_kernel
c4 embed 2 pack_embed
c5 gemm_ffn2 6 linear_lng_kernel<4, 256>
c5 gemm_ffn1 6 linear_tc_kernel<2, 256, 2>
c5 attention 6 attn_tc3_kernel
c5 embed 2 pack_embed}
LIST
