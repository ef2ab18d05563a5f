cd $GRAFT_REPO_ROOT
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_GEMM_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null
python - <<'PY'
import sys; sys.path.insert(0,'.')
import torch, paper_conf_icpp_fuc0z22_b200 as tcb
for K in (512, 2048):
    M,N=32768,512
    A=torch.randn(M,K,device='cuda').bfloat16(); W=(torch.randn(N,K,device='cuda')*0.02).bfloat16(); b=torch.zeros(N,device='cuda')
    R=torch.randn(M,N,device='cuda').bfloat16(); g=torch.ones(N,device='cuda'); be=torch.zeros(N,device='cuda')
    for _ in range(2): tcb.op_linear_ln(A,W,b,R,g,be,1e-5)
    torch.cuda.synchronize()
    print('K',K, flush=True)
    tcb.op_linear_ln(A,W,b,R,g,be,1e-5); torch.cuda.synchronize()
    print('endK',K, flush=True)
PY
