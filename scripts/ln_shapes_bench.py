"""Fused GEMM + bias + residual + LayerNorm (tcb_op_linear_ln) at the encoder's W_O / FFN2
shapes, CUDA-graph replayed (20 calls per replay, L2 warm as in the forward where A was just
written by the previous kernel).  One JSON line per shape: {"workload": "d<d>_k<K>", "us": ...}.
Usage: python scripts/ln_shapes_bench.py [d,K ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_fuc0z22_b200 as tcb

shapes = [tuple(int(v) for v in a.split(",")) for a in sys.argv[1:]] or \
    [(512, 512), (512, 2048), (768, 768), (768, 3072), (1024, 1024), (1024, 4096)]
M = 32768
for d, K in shapes:
    A = (torch.randn(M, K, device="cuda") * 0.5).to(torch.bfloat16)
    W = (torch.randn(d, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
    bias = torch.zeros(d, device="cuda"); g = torch.ones(d, device="cuda"); be = torch.zeros(d, device="cuda")
    R = torch.randn(M, d, device="cuda").to(torch.bfloat16)
    seg = torch.zeros(M, dtype=torch.int32, device="cuda")
    Y = torch.empty(M, d, device="cuda", dtype=torch.bfloat16)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            tcb.op_linear_ln(A, W, bias, R, g, be, 1e-5, seg, Y, stream=s)
    s.synchronize()
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr, stream=s):
        for _ in range(20):
            tcb.op_linear_ln(A, W, bias, R, g, be, 1e-5, seg, Y, stream=s)
    gr.replay(); torch.cuda.synchronize()
    best = 1e9
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s); gr.replay(); b.record(s); s.synchronize()
        best = min(best, a.elapsed_time(b) / 20 * 1e3)
    print(json.dumps({"workload": f"d{d}_k{K}", "us": best,
                      "tflops": 2.0 * M * d * K / best / 1e6}), flush=True)
