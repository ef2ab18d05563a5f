"""GEMM op timing at full SM clock: one launch per iteration between an L2 flush and a 3 ms
idle gap (so the power controller never lowers the clock), CUDA events around the launch only.
Usage: [TCB_GEMM_VARIANT=...] python gemm_fullclock.py"""
import os, sys, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))))
import numpy as np, torch
import paper_conf_icpp_fuc0z22_b200 as tcb

SHAPES = [(32768, 2048, 512, "bias_relu"), (32768, 1536, 512, "bias"), (32768, 3072, 768, "bias_gelu"),
          (32768, 4096, 1024, "bias_gelu")]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for M, N, K, epi in SHAPES:
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    W = (torch.randn(N, K, device="cuda") * 0.02).to(torch.bfloat16)
    b = torch.zeros(N, device="cuda")
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    for _ in range(3): tcb.op_linear(A, W, b, None, epi, out)
    ts = []
    for _ in range(30):
        flush.zero_()
        torch.cuda.synchronize()
        time.sleep(0.003)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); tcb.op_linear(A, W, b, None, epi, out); e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    us = float(np.median(ts)) * 1e3
    print(json.dumps({"M": M, "N": N, "K": K, "epi": epi, "variant": os.environ.get("TCB_GEMM_VARIANT", "default"),
                      "us": us, "tflops": 2.0 * M * N * K / us / 1e6}), flush=True)
