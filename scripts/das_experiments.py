"""§8(f) f2: the online scheduler feeding the B200 encoder (Fig. 9/10, 15, 16-style runs).

The paper (§6.2) serves Poisson request streams (lengths N(20, var) clipped to
[3, 100], R19) and reports total utility (sum of 1/l over requests answered by their
deadline, Eq. (9)), serving throughput, the utility of DAS vs SJF / FCFS / DEF for several
batch sizes, length variances and row lengths (Fig. 15), and the DAS running time relative
to one batch (Fig. 16).  Its V100 rates (40-1500 req/s) do not transfer: here every rate is
a multiple of the measured capacity C of the configuration on this GPU
(C = requests per full batch / full-batch device time).  Deadlines are not specified in the
paper (reading R29): d_n = a_n + U(1, 10) * tau, tau = the full-batch device time.

Every run goes through paper_conf_icpp_fuc0z22_b200.serve.Server (C++ scheduler + CUDA-
graph replay of the encoder per time slot).  One JSON line per run.
Usage: python scripts/das_experiments.py [e1|e7|c5|deadlines|overlap|all] [slots]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import paper_conf_icpp_fuc0z22_b200 as tcb
from paper_conf_icpp_fuc0z22_b200.serve import Server
import tcb_workload as wl

POLICIES = ("das", "sjf", "fcfs", "def")


def lengths_normal(n, var, seed):
    rng = np.random.default_rng(seed)
    return np.clip(np.rint(rng.normal(20.0, np.sqrt(var), size=n)), 3, 100).astype(np.int32)


def full_batch_ms(enc, lengths, B, L):
    """Device time of one full B x L batch (First-Fit rows) under CUDA-graph replay."""
    plan = tcb.tcb_pack(lengths, L, B)
    st = torch.from_numpy(plan.segtab()).cuda()
    ids = torch.zeros(int(plan.info["total_tokens"]), dtype=torch.int32, device="cuda")
    rows = enc.alloc_rows(plan.num_slots)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(2):
            enc.encoder_forward(plan, st, ids, rows, stream=s)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        enc.encoder_forward(plan, st, ids, rows, stream=s)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(10):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    per_batch = plan.info["num_placed"]
    return a.elapsed_time(b) / 10, per_batch


# deadline models (the paper gives none, reading R29): budget in units of tau = full-batch time
DEADLINES = {
    "u1_10": lambda rng, l, n: rng.uniform(1.0, 10.0, size=n),          # R29 (default)
    "u1_3": lambda rng, l, n: rng.uniform(1.0, 3.0, size=n),            # tight
    "const3": lambda rng, l, n: np.full(n, 3.0),                        # one SLA for all
    "len": lambda rng, l, n: 1.0 + 9.0 * l / 100.0,                     # budget grows with length
    "inv_len": lambda rng, l, n: 1.0 + 9.0 * (1.0 - l / 100.0),         # short = interactive
}


def run(enc, model, policy, B, L, rate_mult, var, slots, seed, dist=None, overlap=False,
        deadlines="u1_10"):
    probe = lengths_normal(20000, var, seed + 7) if dist is None else \
        np.minimum(wl.draw_lengths(dist, 20000, seed + 7), L).astype(np.int32)
    tau_ms, per_batch = full_batch_ms(enc, probe, B, L)
    cap = per_batch / (tau_ms / 1e3)                 # requests/s at full batches
    rate = rate_mult * cap
    horizon = slots * tau_ms / 1e3
    n = int(rate * horizon * 1.1) + 16
    rng = np.random.default_rng(seed)
    arrival = np.cumsum(rng.exponential(1.0 / rate, size=n))
    lengths = lengths_normal(n, var, seed + 1) if dist is None else \
        np.minimum(wl.draw_lengths(dist, n, seed + 1), L).astype(np.int32)
    deadline = arrival + DEADLINES[deadlines](rng, lengths, n) * (tau_ms / 1e3)
    offs = np.concatenate([[0], np.cumsum(lengths)])[:-1].astype(np.int64)
    ids = wl.draw_token_ids(int(lengths.sum()), model.vocab, seed + 2)
    srv = Server(enc, policy, B, L, overlap=overlap)
    res = srv.run(lengths, arrival, deadline, ids, offs, horizon)
    res.update({"model": model.name, "rate_x_capacity": rate_mult, "rate_req_s": rate,
                "capacity_req_s": cap, "full_batch_ms": tau_ms, "length_var": var,
                "dist": dist or f"normal(20,{var})", "slots_target": slots, "deadlines": deadlines})
    print(json.dumps(res), flush=True)
    return res


def main():
    what = sys.argv[1] if len(sys.argv) > 1 else "all"
    slots = int(sys.argv[2]) if len(sys.argv) > 2 else 800
    base = wl.MODELS["transformer-base"]
    enc = tcb.Encoder(base, wl.draw_weights(base, 60), wl.weight_names(base))
    if what in ("e1", "all"):          # Fig. 9 / 10 / 16: utility, throughput, overhead vs rate
        for rm in (0.25, 0.5, 0.75, 1.0, 1.5, 2.0, 3.0):
            for pol in POLICIES:
                run(enc, base, pol, 64, 128, rm, 20, slots, 100)
    if what in ("e7", "all"):          # Fig. 15 (a) batch size, (b) variance, (c) row length
        for B in (5, 10, 16):
            for pol in POLICIES:
                run(enc, base, pol, B, 128, 2.0, 20, slots, 200)
        for var in (10, 50, 100):
            for pol in POLICIES:
                run(enc, base, pol, 16, 128, 2.0, var, slots, 300)
        for L in (104, 200, 304):
            for pol in POLICIES:
                run(enc, base, pol, 16, L, 2.0, 20, slots, 400)
    if what == "deadlines":            # DAS vs SJF under other deadline models (R29 is a guess)
        for dl in DEADLINES:
            for B, rm in ((16, 2.0), (64, 1.0), (64, 2.0)):
                for pol in ("das", "sjf", "fcfs"):
                    run(enc, base, pol, B, 128, rm, 50, slots, 600, deadlines=dl)
    if what == "overlap":              # serial vs pipelined scheduler + GPU (Server overlap)
        for rm in (0.5, 1.0, 2.0, 3.0):
            for pol in ("das", "fcfs"):
                for ov in (False, True):
                    run(enc, base, pol, 64, 128, rm, 20, slots, 100, overlap=ov)
    if what in ("c5", "all"):          # C5: Transformer-big encoder, WMT-like, 128 x 256
        big = wl.MODELS["transformer-big"]
        enc_big = tcb.Encoder(big, wl.draw_weights(big, 42), wl.weight_names(big))
        for rm in (0.5, 1.0, 2.0):
            for pol in ("das", "fcfs"):
                run(enc_big, big, pol, 128, 256, rm, 0, max(200, slots // 4), 500, dist="wmt")


if __name__ == "__main__":
    main()
