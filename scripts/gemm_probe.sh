cd $GRAFT_REPO_ROOT
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_GEMM_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > /dev/null
python - <<'PY'
import sys; sys.path.insert(0,'.')
import torch, paper_conf_icpp_fuc0z22_b200 as tcb
for (M,N,K) in [(32768,1536,512),(8192,8192,8192),(32768,512,2048)]:
    A=torch.randn(M,K,device='cuda').bfloat16(); W=(torch.randn(N,K,device='cuda')*0.02).bfloat16(); b=torch.zeros(N,device='cuda')
    R=torch.randn(M,N,device='cuda').bfloat16()
    epi = 'bias_residual' if N==512 else 'bias'
    for _ in range(2): tcb.op_linear(A,W,b,R,epi)
    torch.cuda.synchronize()
    print('shape',M,N,K, flush=True)
    tcb.op_linear(A,W,b,R,epi); torch.cuda.synchronize()
PY
