"""A/B timing of tcb_op_linear_ln: python scripts/ln_ab.py [libA.so libB.so ...] (default: libtcb.so).
Each library is loaded in a fresh subprocess; times are per call inside a CUDA graph."""
import json, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

CHILD = r'''
import sys, json, torch
sys.path.insert(0, ".")
import paper_conf_icpp_fuc0z22_b200._lib as L
L.SO_PATH = sys.argv[1]
import paper_conf_icpp_fuc0z22_b200 as tcb
def t_us(fn, it=40):
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3): fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(it): fn()
    g.replay(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); g.replay(); b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it * 1e3
for M, K in [(32768, 512), (32768, 2048), (16384, 512), (16384, 2048)]:
    N = 512
    A = torch.randn(M, K, device="cuda").bfloat16(); W = (torch.randn(N, K, device="cuda") * 0.02).bfloat16()
    bb = torch.zeros(N, device="cuda"); R = torch.randn(M, N, device="cuda").bfloat16()
    g = torch.ones(N, device="cuda"); be = torch.zeros(N, device="cuda")
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    us = t_us(lambda: tcb.op_linear_ln(A, W, bb, R, g, be, 1e-5, None, out, stream=torch.cuda.current_stream()))
    print(json.dumps({"lib": sys.argv[1].split("/")[-1], "M": M, "K": K, "us": round(us, 2),
                      "tflops": round(2 * M * N * K / us / 1e6, 1)}), flush=True)
'''
libs = sys.argv[1:] or ["paper_conf_icpp_fuc0z22_b200/libtcb.so"]
for lib in libs:
    subprocess.run([sys.executable, "-c", CHILD, lib], check=False)
