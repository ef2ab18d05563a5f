# in-kernel clock64 probe of linear_ln_kernel (d = 512 W_O + LN1, K = 512) -> per-role cycle split
cd $GRAFT_REPO_ROOT; T=gpurun_out/${TAG:-lnprobe}; mkdir -p $T
sed -i 's/FLAGS = \["-O3"/FLAGS = ["-DTCB_LN_PROBE", "-O3"/' paper_conf_icpp_fuc0z22_b200/_build.py
python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build(force=True)" > $T/build.log 2>&1; echo build rc $?
python - <<'PY' 2>&1 | tee $T/probe.txt
import sys; sys.path.insert(0,'.')
import torch, paper_conf_icpp_fuc0z22_b200 as tcb
M,N,K=32768,512,512
A=torch.randn(M,K,device='cuda').bfloat16(); W=(torch.randn(N,K,device='cuda')*0.02).bfloat16(); b=torch.zeros(N,device='cuda')
R=torch.randn(M,N,device='cuda').bfloat16(); g=torch.ones(N,device='cuda'); be=torch.zeros(N,device='cuda')
for _ in range(3): tcb.op_linear_ln(A,W,b,R,g,be,1e-5)
torch.cuda.synchronize()
print('=== probe run', flush=True)
tcb.op_linear_ln(A,W,b,R,g,be,1e-5); torch.cuda.synchronize()
print('=== end', flush=True)
PY
