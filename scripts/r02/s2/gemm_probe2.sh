# clock64 probe of linear_tc_kernel: MMA warp (wait operands / wait accumulator free / issue)
# and epilogue warps (wait accumulator full / work per tile) on the encoder GEMM shapes
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-gprobe}; mkdir -p $T
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_GEMM_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > $T/build.log 2>&1; echo build rc $?
timeout 120 python - <<'PY' 2>&1 | tee $T/probe.txt
import sys; sys.path.insert(0,'.')
import torch, paper_conf_icpp_fuc0z22_b200 as tcb
for (M,N,K,epi) in [(32768,2048,512,'bias_relu'),(32768,1536,512,'bias'),(32768,4096,1024,'bias_gelu'),(8192,8192,8192,'bias')]:
    A=torch.randn(M,K,device='cuda').bfloat16(); W=(torch.randn(N,K,device='cuda')*0.02).bfloat16(); b=torch.zeros(N,device='cuda')
    for _ in range(2): tcb.op_linear(A,W,b,None,epi)
    torch.cuda.synchronize()
    print('shape',M,N,K,epi, flush=True)
    tcb.op_linear(A,W,b,None,epi); torch.cuda.synchronize()
PY
