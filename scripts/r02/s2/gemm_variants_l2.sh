# Is the tcgen05 GEMM bound by L2 -> SM bytes?  Same shapes, tile shapes with 1x / 1.5x the L2
# bytes per MAC (cg2_256: 256x256 pair tiles; cg2_128 / cg1_256: 256x128 / 128x256), plus ncu L2
# throughput of the default on the C2 FFN1 shape.
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-l2}; mkdir -p $T
python -c "import __graft_entry__ as g; g.build()" > $T/build.log 2>&1; echo build rc $?
export SHAPES="32768,2048,512,bias_relu 32768,1536,512,bias 32768,4096,1024,bias_gelu 8192,8192,8192,bias"
for v in default cg2_128 cg1_256; do
  if [ $v = default ]; then timeout 120 python scripts/gemm_bench.py; else TCB_GEMM_VARIANT=$v timeout 120 python scripts/gemm_bench.py; fi
done 2>&1 | tee $T/variants.jsonl
