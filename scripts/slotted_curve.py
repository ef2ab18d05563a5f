"""§8(f) f1: slotted vs pure ConcatBatching on B200 (the Fig. 13/14-style curve).

The paper (§6.2.3) fixes the batch size B (10, then 32) and reports the
speedup of the average batch inference time of slotted ConcatBatching over pure
ConcatBatching (1 slot) for 1, 2, 4, 5, 7, 10, 20 slots: at most 1.18x (B = 10) and 2.31x
(B = 32, 7 slots).  Here: Transformer-base encoder (C2's model, the paper's encoder size),
request stream from the paper's length distribution N(20, 20) clipped to [3, 100] (R19),
B rows x L words; for every slot count s the first batch of the stream is packed with
tcb_pack_slotted(z = L // s) (s = 1 is pure First-Fit) and its forward is timed under
CUDA-graph replay.  Prints one JSON line per (L, B, s): batch time, speedup over s = 1,
placed tokens, tokens/s, padding, attention KV tiles visited, attention-class device time.

Usage: python scripts/slotted_curve.py [L ...]     (default L = 256 512)
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import paper_conf_icpp_fuc0z22_b200 as tcb
import tcb_workload as wl

SLOTS = (1, 2, 4, 5, 7, 10, 20)


def time_forward(enc, plan, d_ids, reps=20):
    st = torch.from_numpy(plan.segtab()).cuda()
    rows = enc.alloc_rows(plan.num_slots)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            enc.encoder_forward(plan, st, d_ids, rows, stream=s)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        enc.encoder_forward(plan, st, d_ids, rows, stream=s)
    g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / reps
    tcb.profile_enable(True)
    with torch.cuda.stream(s):
        enc.encoder_forward(plan, st, d_ids, rows, stream=s)
    s.synchronize()
    prof = tcb.profile_collect()
    tcb.profile_enable(False)
    return ms, prof["attention"][0]


def main():
    Ls = [int(x) for x in sys.argv[1:]] or [256, 512]
    model = wl.MODELS["transformer-base"]
    enc = tcb.Encoder(model, wl.draw_weights(model, 52), wl.weight_names(model))
    lengths_all = wl.draw_lengths("paper_normal_20", 200000, 50).astype(np.int32)
    cu = np.concatenate([[0], np.cumsum(lengths_all)])
    ids_all = wl.draw_token_ids(int(cu[-1]), model.vocab, 51)
    for L in Ls:
        for B in (10, 32, 256):
            base = None
            for s in SLOTS:
                z = L // s
                if z < 8:
                    continue
                plan = tcb.tcb_pack_slotted(lengths_all[:B * L // 3], L, z if s > 1 else L, B)
                a = plan.arrays()
                placed = np.flatnonzero(a["req_row"] >= 0)
                # the segment table indexes token ids by request order over ALL requests
                d_ids = torch.from_numpy(ids_all[:cu[B * L // 3]]).cuda()
                ms, attn_ms = time_forward(enc, plan, d_ids)
                i = plan.info
                if base is None:
                    base = ms
                print(json.dumps({
                    "L": L, "B": B, "slots": s, "slot_len": i["slot_len"],
                    "rows": i["num_rows"], "requests_placed": int(len(placed)),
                    "placed_tokens": i["placed_tokens"],
                    "padding_fraction": round(1 - i["placed_tokens"] / i["num_slots"], 4),
                    "batch_ms": round(ms, 4), "speedup_vs_1slot": round(base / ms, 3),
                    "tokens_per_s": round(i["placed_tokens"] / (ms / 1e3)),
                    "attention_ms": round(attn_ms, 4),
                    "kv_tiles_visited": i["kv_tiles_visited"], "kv_tiles_dense": i["kv_tiles_dense"],
                    "useful_score_elems": i["useful_score_elems"]}), flush=True)


if __name__ == "__main__":
    main()
