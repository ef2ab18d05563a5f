"""Microbenchmark of the segment-masked attention kernel (tcb_op_attention) on the packed
layouts of the BASELINE workloads; prints time, useful-flop rate and HBM-byte rate."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb

def t_ms(fn, it=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it

for key in sys.argv[1:] or ["c2", "c3", "c5"]:
    w = wl.WORKLOADS[key]
    lengths = wl.lengths_filling(w.lengths, w.rows, w.row_len, w.seeds[0])
    plan = tcb.tcb_pack(lengths, w.row_len, w.rows)
    M, d, h = plan.num_slots, w.model.d_model, w.model.num_heads
    qkv = (torch.randn(M, 3 * d, device="cuda") * 0.5).to(torch.bfloat16)
    seg = torch.from_numpy(plan.arrays()["segment_ids"]).cuda()
    st = torch.from_numpy(plan.segtab()).cuda()
    out = torch.empty(M, d, device="cuda", dtype=torch.bfloat16)
    ms = t_ms(lambda: tcb.op_attention(qkv, seg, st, h, out))
    useful = plan.info["useful_score_elems"]
    byts = M * 3 * d * 2 + M * d * 2
    print(json.dumps({"workload": key, "us": ms * 1e3, "useful_tflops": 4.0 * d * useful / ms / 1e9,
                      "gbps": byts / ms / 1e6, "executed_frac_of_dense": plan.info["executed_score_elems"] / (plan.info["num_rows"] * w.row_len ** 2)}), flush=True)
