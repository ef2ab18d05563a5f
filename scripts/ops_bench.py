"""Graph-timed microbenchmarks of the HBM-bound kernels (pack_embed, layernorm, unpack) on a
BASELINE workload's packed layout; prints us and GB/s of algorithmic bytes."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb


def t_ms(fn, it=40):
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


for key in sys.argv[1:] or ["c2", "c3"]:
    w = wl.WORKLOADS[key]
    m = w.model
    lengths, ids, weights = wl.workload_inputs(key)
    enc = tcb.Encoder(m, weights, wl.weight_names(m))
    plan = tcb.tcb_pack(lengths, w.row_len, w.rows)
    M, d, T = plan.num_slots, m.d_model, plan.info["placed_tokens"]
    st = torch.from_numpy(plan.segtab()).cuda()
    d_ids = torch.from_numpy(ids).cuda()
    rows = enc.alloc_rows(M)
    seg = torch.empty(M, dtype=torch.int32, device="cuda")
    out = torch.empty(plan.info["total_tokens"], d, dtype=enc.dtype, device="cuda")
    ms = t_ms(lambda s: enc.embed(plan, st, d_ids, rows, seg, None, stream=s))
    print(json.dumps({"workload": key, "kernel": "pack_embed", "us": ms * 1e3,
                      "gbps": (T * (4 + 2 * d) + M * (2 * d + 4)) / ms / 1e6}), flush=True)
    ms = t_ms(lambda s: enc.unpack(plan, st, rows, out, stream=s))
    print(json.dumps({"workload": key, "kernel": "unpack", "us": ms * 1e3,
                      "gbps": 4 * T * d / ms / 1e6}), flush=True)
    g = torch.ones(d, device="cuda"); b = torch.zeros(d, device="cuda")
    y = torch.empty_like(rows)
    ms = t_ms(lambda s: tcb.op_layernorm(rows, g, b, 1e-5, seg, y, stream=s))
    print(json.dumps({"workload": key, "kernel": "layernorm", "us": ms * 1e3,
                      "gbps": 4 * M * d / ms / 1e6}), flush=True)
