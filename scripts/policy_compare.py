"""BASELINE config 3: ConcatBatching vs NaiveBatching vs length-sorted batching on the SAME
request stream (BERT-base, DIA-like lengths, B = 64 rows per forward).

* concat       : First-Fit into rows of L = 512 (pure ConcatBatching, Fig. 1(c))
* naive        : B requests per forward, one per row, padded to the batch maximum (TNB,
                 Fig. 1(a); reading R17: pad keys masked)
* length_sorted: windows of 16*B requests sorted by length, then batches of B, each padded to
                 its maximum (TurboTransformers-like; reading R18)

Every forward runs through the same C ABI (tcb_encoder_forward); per-forward device time is
taken with CUDA events; the metric is non-pad tokens / total device time.  Prints one JSON
line per policy.  Usage: python scripts/policy_compare.py [workload] [num_requests]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import paper_conf_icpp_fuc0z22_b200 as tcb
import tcb_workload as wl


def batches(policy, lengths, B, L):
    n = len(lengths)
    idx = np.arange(n)
    if policy == "concat":
        # stream prefix order; First-Fit with a B-row cap, deferred requests go to the next
        pending = list(idx)
        while pending:
            plan = tcb.tcb_pack(lengths[pending], L, B, "first_fit")
            rows = plan.arrays()["req_row"]
            placed = [pending[i] for i in range(len(pending)) if rows[i] >= 0]
            yield np.array(placed), L, "first_fit"
            pending = [pending[i] for i in range(len(pending)) if rows[i] < 0]
    elif policy == "naive":
        for s in range(0, n, B):
            sel = idx[s:s + B]
            yield sel, int(-(-lengths[sel].max() // 8) * 8), "naive"
    elif policy == "length_sorted":
        W = 16 * B
        for w0 in range(0, n, W):
            win = idx[w0:w0 + W]
            win = win[np.argsort(lengths[win], kind="stable")]
            for s in range(0, len(win), B):
                sel = win[s:s + B]
                yield sel, int(-(-lengths[sel].max() // 8) * 8), "naive"


def main():
    key = sys.argv[1] if len(sys.argv) > 1 else "c3"
    nreq = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
    w = wl.WORKLOADS[key]
    m = w.model
    lengths = np.minimum(wl.draw_lengths(w.lengths, nreq, w.seeds[0]), w.row_len).astype(np.int32)
    cu = np.concatenate([[0], np.cumsum(lengths)])
    ids_all = wl.draw_token_ids(int(cu[-1]), m.vocab, w.seeds[1])
    enc = tcb.Encoder(m, wl.draw_weights(m, w.seeds[2]), wl.weight_names(m))
    for policy in ("concat", "naive", "length_sorted"):
        total_ms, tokens, slots, forwards = 0.0, 0, 0, 0
        for sel, L, pol in batches(policy, lengths, w.rows, w.row_len):
            ls = lengths[sel]
            ids = np.concatenate([ids_all[cu[i]:cu[i + 1]] for i in sel])
            plan = tcb.tcb_pack(ls, L, w.rows, pol)
            st = torch.from_numpy(plan.segtab()).cuda()
            d_ids = torch.from_numpy(ids).cuda()
            rows = enc.alloc_rows(plan.num_slots)
            enc.encoder_forward(plan, st, d_ids, rows)           # warm (descriptor cache)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            enc.encoder_forward(plan, st, d_ids, rows)
            b.record()
            torch.cuda.synchronize()
            total_ms += a.elapsed_time(b)
            tokens += plan.info["placed_tokens"]
            slots += plan.info["num_slots"]
            forwards += 1
        print(json.dumps({"workload": w.name, "policy": policy, "requests": nreq,
                          "non_pad_tokens": tokens, "forwards": forwards,
                          "padding_fraction": 1 - tokens / slots,
                          "device_ms": total_ms, "tokens_per_s": tokens / (total_ms / 1e3)}),
              flush=True)


if __name__ == "__main__":
    main()
