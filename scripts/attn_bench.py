"""Microbenchmark of the segment-masked attention kernel (tcb_op_attention) on the packed
layouts of the BASELINE workloads; prints time, useful-flop rate and HBM-byte rate.  The op
call (counter reset + kernel) is captured once in a CUDA graph and replayed, so host overhead
is not timed; the L2 is flushed between replays (QKV is read from HBM as in the forward)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb


def t_us(fn, it=20):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3): fn()
        s.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            fn()
        ts = []
        for _ in range(it):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s); g.replay(); b.record(s)
            ts.append((a, b))
        s.synchronize()
    return float(np.median([a.elapsed_time(b) for a, b in ts])) * 1e3


if __name__ == "__main__":
    for key in sys.argv[1:] or ["c2", "c3", "c5"]:
        w = wl.WORKLOADS[key]
        lengths = wl.lengths_filling(w.lengths, w.rows, w.row_len, w.seeds[0])
        plan = tcb.tcb_pack(lengths, w.row_len, w.rows)
        M, d, h = plan.num_slots, w.model.d_model, w.model.num_heads
        qkv = (torch.randn(M, 3 * d, device="cuda") * 0.5).to(torch.bfloat16)
        seg = torch.from_numpy(plan.arrays()["segment_ids"]).cuda()
        st = torch.from_numpy(plan.segtab()).cuda()
        out = torch.empty(M, d, device="cuda", dtype=torch.bfloat16)
        us = t_us(lambda: tcb.op_attention(qkv, seg, st, h, out))
        info = plan.info
        byts = M * 3 * d * 2 + M * d * 2
        print(json.dumps({"workload": key, "impl": os.environ.get("TCB_ATTN", "v2"), "us": us,
                          "useful_tflops": 4.0 * d * info["useful_score_elems"] / us / 1e6,
                          "gbps": byts / us / 1e3,
                          "executed_frac_of_dense": info["executed_score_elems"] / (info["num_rows"] * w.row_len ** 2),
                          "softmax_frac_of_executed": info["softmax_score_elems"] / max(info["executed_score_elems"], 1),
                          "chunks_per_head": info["executed_score_elems"] // (128 * 128)}), flush=True)
