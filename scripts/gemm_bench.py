"""Microbenchmark: tcb tcgen05 GEMM (tcb_op_linear) vs torch.matmul (cuBLAS) on the encoder's
GEMM shapes and a square reference shape.  Usage: python scripts/gemm_bench.py [variant...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_fuc0z22_b200 as tcb

SHAPES = [(32768, 1536, 512, "bias"), (32768, 512, 512, "bias_residual"),
          (32768, 2048, 512, "bias_relu"), (32768, 512, 2048, "bias_residual"),
          (32768, 2304, 768, "bias"), (32768, 3072, 768, "bias_gelu"),
          (32768, 3072, 1024, "bias"), (32768, 4096, 1024, "bias_gelu"),
          (8192, 8192, 8192, "bias")]
if os.environ.get("SHAPES"):
    SHAPES = [tuple(int(x) for x in s.split(",")[:3]) + (s.split(",")[3],) for s in os.environ["SHAPES"].split()]

def t_ms(fn, it=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it

res = []
for M, N, K, epi in SHAPES:
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (torch.randn(N, K, device="cuda") * 0.02).to(torch.bfloat16)
    b = torch.zeros(N, device="cuda")
    R = torch.randn(M, N, device="cuda").to(torch.bfloat16) if epi == "bias_residual" else None
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    ours = t_ms(lambda: tcb.op_linear(A, W, b, R, epi, out))
    cub = t_ms(lambda: torch.matmul(A, W.t(), out=out))
    fl = 2.0 * M * N * K
    res.append({"M": M, "N": N, "K": K, "epi": epi, "variant": os.environ.get("TCB_GEMM_VARIANT", "default"),
                "ours_tflops": fl / ours / 1e9, "cublas_tflops": fl / cub / 1e9})
    print(json.dumps(res[-1]), flush=True)
