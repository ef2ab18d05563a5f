"""FFN1 shapes (C3: N=3072, K=768; C4: N=4096, K=1024; M=32768) under each epilogue, to price
the activation epilogue (tcb_op_linear); prints TFLOP/s per (shape, epilogue)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_fuc0z22_b200 as tcb


def t_ms(fn, it=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it


for M, N, K in [(32768, 3072, 768), (32768, 4096, 1024), (32768, 2048, 512)]:
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (torch.randn(N, K, device="cuda") * 0.02).to(torch.bfloat16)
    b = torch.zeros(N, device="cuda")
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    for epi in ["bias", "bias_relu", "bias_gelu"]:
        ms = t_ms(lambda: tcb.op_linear(A, W, b, None, epi, out))
        print(json.dumps({"M": M, "N": N, "K": K, "epi": epi, "us": ms * 1e3,
                          "tflops": 2.0 * M * N * K / ms / 1e9,
                          "tag": os.environ.get("TAG", "")}), flush=True)
