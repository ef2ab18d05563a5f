"""Does splitting a step's rows into two halves on two streams (one CUDA graph, fork/join)
beat one forward over all rows?  The halves' kernels can fill each other's wave tails and
prologues.  Prints ms per step (L2 flushed before each) for: one 2B-row forward, and two B-row
forwards on two streams.  Usage: python two_stream_halves.py c2 [c3 ...]"""
import os, sys, json
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.path.insert(0, ROOT)
import numpy as np, torch
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb

dev = torch.device("cuda:0")
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)


def setup(enc, key, rows, seed_off):
    w = wl.WORKLOADS[key]
    lengths = wl.lengths_filling(w.lengths, rows, w.row_len, w.seeds[0] + seed_off, 0.995)
    ids = wl.draw_token_ids(int(lengths.sum()), w.model.vocab, w.seeds[1] + seed_off)
    plan = tcb.tcb_pack(lengths, w.row_len, rows)
    st = torch.from_numpy(plan.segtab()).to(dev)
    d_ids = torch.from_numpy(ids).to(dev)
    r = enc.alloc_rows(plan.info["num_slots"])
    out = torch.empty((plan.info["total_tokens"], w.model.d_model), dtype=enc.dtype, device=dev)
    return plan, st, d_ids, r, out


def time_graph(g, s, it=20):
    ts = []
    with torch.cuda.stream(s):          # replay() launches on the current stream
        for _ in range(3):
            g.replay()
        torch.cuda.synchronize()
        for _ in range(it):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s); g.replay(); b.record(s)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
    return float(np.median(ts))


for key in sys.argv[1:] or ["c2"]:
    w = wl.WORKLOADS[key]
    names = wl.weight_names(w.model)
    enc = tcb.Encoder(w.model, wl.draw_weights(w.model, w.seeds[2]), names)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    full = setup(enc, key, w.rows, 0)
    half_a = setup(enc, key, w.rows // 2, 0)
    half_b = setup(enc, key, w.rows // 2, 500)
    enc2 = tcb.Encoder(w.model, None, names, tensors=enc.tensors) if hasattr(enc, "tensors") else enc

    def fwd(e, x, s):
        plan, st, d_ids, r, out = x
        e.encoder_forward(plan, st, d_ids, r, stream=s)
        e.unpack(plan, st, r, out, stream=s)

    with torch.cuda.stream(s1):
        fwd(enc, full, s1)
    torch.cuda.synchronize()
    g1 = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g1, stream=s1):
        fwd(enc, full, s1)
    t1 = time_graph(g1, s1)

    with torch.cuda.stream(s1):
        fwd(enc, half_a, s1)
        fwd(enc2, half_b, s1)
    torch.cuda.synchronize()
    g2 = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g2, stream=s1):
        e0 = torch.cuda.Event()
        e0.record(s1)
        s2.wait_event(e0)
        fwd(enc, half_a, s1)
        fwd(enc2, half_b, s2)
        e1 = torch.cuda.Event()
        e1.record(s2)
        s1.wait_event(e1)
    t2 = time_graph(g2, s1)
    ta = full[0].info["placed_tokens"]
    tb = half_a[0].info["placed_tokens"] + half_b[0].info["placed_tokens"]
    print(json.dumps({"workload": key, "one_forward_ms": t1, "one_forward_Mtok_s": ta / t1 / 1e3,
                      "two_stream_halves_ms": t2, "two_stream_Mtok_s": tb / t2 / 1e3}), flush=True)
