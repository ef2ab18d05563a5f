cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-fullclock}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
(nvidia-smi --query-gpu=clocks.sm,power.draw --format=csv,noheader -lms 50 > $T/clocks.csv 2>&1 &) ; 
for v in default cg1_256 cg2_128; do
  if [ $v = default ]; then timeout 120 python scripts/r02/s2/gemm_fullclock.py; else TCB_GEMM_VARIANT=$v timeout 120 python scripts/r02/s2/gemm_fullclock.py; fi
done 2>&1 | tee $T/fullclock.jsonl
sort $T/clocks.csv | uniq -c | sort -rn | head -5
