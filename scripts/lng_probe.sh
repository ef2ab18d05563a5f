# linear_lng_kernel (L2-exchange LN GEMM) epilogue phase probe at the C2 FFN2 / C4 FFN2 shapes
cd $GRAFT_REPO_ROOT
TCB_EXTRA_NVCC_FLAGS="-DTCB_LN_PROBE" python -c "import sys; sys.path.insert(0,'paper_conf_icpp_fuc0z22_b200'); import _build; _build.build()" > /dev/null 2>&1
TCB_EXTRA_NVCC_FLAGS="-DTCB_LN_PROBE" python - <<'PY'
import torch, sys
sys.path.insert(0, '.')
import paper_conf_icpp_fuc0z22_b200 as tcb
for (M, K, N) in [(32768, 2048, 512), (32768, 4096, 1024)]:
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (torch.randn(N, K, device="cuda") * 0.02).to(torch.bfloat16)
    b = torch.zeros(N, device="cuda"); g = torch.ones(N, device="cuda"); be = torch.zeros(N, device="cuda")
    R = torch.randn(M, N, device="cuda").to(torch.bfloat16)
    for i in range(2):
        out = tcb.op_linear_ln(A, W, b, R, g, be, 1e-5, None)
        torch.cuda.synchronize()
        print("---", M, K, N, i, flush=True)
PY
