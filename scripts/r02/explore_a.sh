# r02 exploration: where do the K=512 GEMMs and the attention kernel lose time?
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02a/build.log 2>&1; echo build rc $?
timeout 300 python scripts/gemm_bench.py > gpurun_out/r02a/gemm_bench.txt 2>&1; echo gemm_bench rc $?
timeout 300 python scripts/attn_bench.py c2 c3 c4 c5 > gpurun_out/r02a/attn_bench.txt 2>&1; echo attn_bench rc $?
# ncu full capture of the QKV-shape GEMM (op level) with source
cat > /tmp/qkv_once.py <<'PY'
import sys; sys.path.insert(0,'.')
import torch, paper_conf_icpp_fuc0z22_b200 as tcb
M,N,K = [int(x) for x in sys.argv[1:4]]
A=torch.randn(M,K,device='cuda').bfloat16(); W=(torch.randn(N,K,device='cuda')*0.02).bfloat16(); b=torch.zeros(N,device='cuda')
for _ in range(3): tcb.op_linear(A,W,b,None,'bias')
torch.cuda.synchronize()
PY
timeout 300 ncu --set full --clock-control none --import-source on -k regex:linear_tc_kernel -s 2 -c 1 -o gpurun_out/r02a/qkv_c2 python /tmp/qkv_once.py 32768 1536 512 > gpurun_out/r02a/ncu_qkv.log 2>&1; echo ncu qkv rc $?
# instrumented builds: GEMM probe and attention probe
cp paper_conf_icpp_fuc0z22_b200/_build.py /tmp/_build.py.orig
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_GEMM_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1
for s in "32768 1536 512" "32768 2048 512" "8192 8192 8192"; do echo "shape $s"; timeout 120 python /tmp/qkv_once.py $s 2>&1 | grep probe | head -8; done > gpurun_out/r02a/gemm_probe.txt
cp /tmp/_build.py.orig paper_conf_icpp_fuc0z22_b200/_build.py
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_ATTN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null 2>&1
for w in c2 c3 c4; do echo "W $w"; timeout 120 python scripts/attn_bench.py $w 2>&1 | grep -E "tcprobe|workload" | tail -4; done > gpurun_out/r02a/attn_probe.txt
cp /tmp/_build.py.orig paper_conf_icpp_fuc0z22_b200/_build.py
echo done
