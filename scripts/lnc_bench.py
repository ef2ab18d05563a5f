"""Microbenchmark: fused GEMM + bias + residual + LayerNorm (tcb_op_linear_ln) vs the unfused
pair (tcb_op_linear bias_residual + tcb_op_layernorm) at the encoder's W_O / FFN2 shapes."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_fuc0z22_b200 as tcb

def t_ms(fn, it=20):
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3): fn(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(it): fn(s)
    g.replay(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); g.replay(); b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it

M = 32768
for d, K in [(512, 512), (512, 2048), (768, 768), (768, 3072), (1024, 1024), (1024, 4096)]:
    A = (torch.randn(M, K, device="cuda") * 0.5).to(torch.bfloat16)
    W = (torch.randn(d, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
    bias = torch.zeros(d, device="cuda"); g = torch.ones(d, device="cuda"); be = torch.zeros(d, device="cuda")
    R = torch.randn(M, d, device="cuda").to(torch.bfloat16)
    seg = torch.zeros(M, dtype=torch.int32, device="cuda")
    Y = torch.empty(M, d, device="cuda", dtype=torch.bfloat16)
    Z = torch.empty_like(Y)
    fused = t_ms(lambda s: tcb.op_linear_ln(A, W, bias, R, g, be, 1e-5, seg, Y, stream=s))
    def unf(s):
        tcb.op_linear(A, W, bias, R, "bias_residual", out=Z, stream=s)
        tcb.op_layernorm(Z, g, be, 1e-5, seg, Y, stream=s)
    unfused = t_ms(unf)
    fl = 2.0 * M * d * K
    print(json.dumps({"d": d, "K": K, "fused_us": fused * 1e3, "unfused_us": unfused * 1e3,
                      "fused_tflops": fl / fused / 1e9}), flush=True)
