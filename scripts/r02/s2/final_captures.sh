# ncu --set full raw pages (CSV) of the GEMM / LayerNorm-GEMM classes (demangled names carry
# "(int)" casts in this ncu) -> gpurun_out/$TAG/full
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-final3}; mkdir -p $T/full /tmp/reps
python -c "import __graft_entry__ as g; g.build()" > $T/build_caps.log 2>&1 || exit 1
while read -r w c s k; do
  [ -z "$w" ] && continue
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s $s -c 1 -f -o /tmp/reps/${w}_$c env TCB_NO_COOP=1 python bench.py --workload $w --steps 1 --warmup 2 \
    --no-cpu-baseline --no-graph > $T/full/${w}_$c.log 2>&1
  echo "full $w $c rc $?"
  ncu -i /tmp/reps/${w}_$c.ncu-rep --page raw --csv > $T/full/${w}_$c.csv 2>&1
done <<LIST
c2 gemm_qkv 6 linear_tc_kernel<\(int\)2, \(int\)256, \(int\)0>
c2 gemm_ffn1 6 linear_tc_kernel<\(int\)2, \(int\)256, \(int\)2>
c2 gemm_ffn2 6 linear_lng_kernel<\(int\)2, \(bool\)0>
c3 gemm_o 6 linear_lnc_kernel<\(int\)3>
c3 gemm_ffn2 6 linear_lng_kernel<\(int\)3, \(bool\)0>
LIST
wc -c $T/full/*.csv
