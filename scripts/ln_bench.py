"""Microbenchmark of tcb_op_layernorm at the encoder's shapes (GB/s of algorithmic bytes)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_fuc0z22_b200 as tcb

def t_ms(fn, it=50):
    """Device time per call: `it` calls captured in one CUDA graph (no host overhead)."""
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3): fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(it): fn()
    g.replay(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); g.replay(); b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it

for M, d in [(32768, 512), (32768, 768), (32768, 1024)]:
    Z = torch.randn(M, d, device="cuda").to(torch.bfloat16)
    g = torch.ones(d, device="cuda"); b = torch.zeros(d, device="cuda")
    seg = torch.zeros(M, dtype=torch.int32, device="cuda")
    Y = torch.empty_like(Z)
    ms = t_ms(lambda: tcb.op_layernorm(Z, g, b, 1e-5, seg, Y, stream=torch.cuda.current_stream()))
    print(json.dumps({"M": M, "d": d, "us": ms * 1e3, "gbps": 4 * M * d / ms / 1e6}), flush=True)
