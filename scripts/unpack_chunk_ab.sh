# A/B of the unpack kernel's slots per CTA (TCB_UNPACK_CHUNK) and loads per thread per batch (TCB_UNPACK_U).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
B="import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build()"
for v in "16 4" "32 4" "32 8" "64 8" "64 16" "16 4"; do
  set -- $v
  TCB_EXTRA_NVCC_FLAGS="-DTCB_UNPACK_CHUNK=$1 -DTCB_UNPACK_U=$2" python -c "$B" > /dev/null 2>&1
  echo "chunk $1 U $2"; python scripts/ops_bench.py c2 c3 c4 c5 2>&1 | grep unpack
done
