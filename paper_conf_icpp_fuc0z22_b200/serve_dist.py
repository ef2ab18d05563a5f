"""Multi-GPU online serving (BASELINE configs[4]): one Poisson request stream
spread over W ranks (one process per GPU, torchrun), each rank running its own scheduler and
encoder replica.

TCB's service model (§5.1): requests arrive over time; in every time slot the
scheduler (DAS, Alg. 1, or a baseline) picks from the waiting set the batch of B
rows x L words the GPU runs next.  Across GPUs the rows are independent (the mask of Eq. (6)
confines attention to one request), so the stream is split by a dispatcher in front of the
ranks and there is NO per-step collective:

* the global stream is Poisson(lambda) with WMT-like lengths (C5) and deadlines a + U(1,10) tau
  (reading R29); every rank draws the SAME global stream from the seed and keeps the requests
  the dispatcher sends it -- independent thinning with probability 1/W (a seeded uniform draw
  per request), so rank r sees a Poisson(lambda / W) substream and the substreams partition
  the global one (tests/test_dist_cpu.py checks both with gloo, world size 2);
* each rank serves its substream with serve.Server (C++ scheduler + one CUDA-graph replay of
  forward + unpack per slot) on its own GPU, weights broadcast once (dist.broadcast_weights);
* sustained throughput = tokens answered by all ranks / the longest rank's serving time
  (max over ranks of the simulated clock: scheduler host time + device time per slot); the
  only collectives are the one weight broadcast and the final reductions of the counters.
"""
from __future__ import annotations

from typing import Dict, Tuple

import numpy as np


def global_stream(n: int, rate: float, dist: str, max_len: int, tau: float, seed: int):
    """The global request stream: Poisson(rate) arrivals (seconds), lengths from the named
    distribution clipped to max_len, deadlines a + U(1, 10) * tau (R29), request ids 0..n-1."""
    import tcb_workload as wl
    rng = np.random.default_rng(seed)
    arrival = np.cumsum(rng.exponential(1.0 / rate, size=n))
    lengths = np.minimum(wl.draw_lengths(dist, n, seed + 1), max_len).astype(np.int32)
    deadline = arrival + rng.uniform(1.0, 10.0, size=n) * tau
    return arrival, lengths, deadline


def dispatch(n: int, world: int, seed: int) -> np.ndarray:
    """Rank of every request of the global stream: independent thinning, P(rank) = 1/W."""
    rng = np.random.default_rng(seed + 7)
    return np.minimum((rng.random(n) * world).astype(np.int64), world - 1)


def substream(rank: int, world: int, n: int, rate: float, dist: str, max_len: int, tau: float,
              seed: int) -> Dict[str, np.ndarray]:
    """This rank's share of the global stream (global request ids kept)."""
    arrival, lengths, deadline = global_stream(n, rate, dist, max_len, tau, seed)
    mine = np.nonzero(dispatch(n, world, seed) == rank)[0]
    return {"id": mine, "arrival": arrival[mine], "length": lengths[mine],
            "deadline": deadline[mine]}


def reduce_results(res: Dict[str, float], world: int) -> Dict[str, float]:
    """Whole-job counters: sums of tokens / responses / utility / expiries, max of the serving
    clock (the job lasts as long as its slowest rank).  One all_reduce each."""
    import torch
    import torch.distributed as dist
    sums = torch.tensor([res["tokens"], res["scheduled"], res["utility"], res["expired"],
                         res["requests"], res["batches"]], dtype=torch.float64)
    mx = torch.tensor([res["sim_seconds"], res["batch_ms"], res["sched_ms"]], dtype=torch.float64)
    if world > 1 and dist.is_initialized():
        dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
        sums, mx = sums.to(dev), mx.to(dev)
        dist.all_reduce(sums, op=dist.ReduceOp.SUM)
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        sums, mx = sums.cpu(), mx.cpu()
    s, m = sums.tolist(), mx.tolist()
    return {"tokens": s[0], "responses": s[1], "utility": s[2], "expired": s[3],
            "requests": s[4], "batches": s[5], "seconds": m[0], "max_batch_ms": m[1],
            "max_sched_ms": m[2], "tokens_per_s": s[0] / max(m[0], 1e-12),
            "responses_per_s": s[1] / max(m[0], 1e-12)}


def serve_rank(encoder, sub: Dict[str, np.ndarray], vocab: int, B: int, L: int, policy: str,
               horizon: float, seed: int, overlap: bool = True) -> Dict[str, float]:
    """Serve this rank's substream on its GPU until its clock passes ``horizon`` seconds."""
    import tcb_workload as wl
    from .serve import Server
    lengths = sub["length"].astype(np.int32)
    tok_off = np.concatenate([[0], np.cumsum(lengths.astype(np.int64))[:-1]])
    token_ids = wl.draw_token_ids(int(lengths.sum()), vocab, seed)
    srv = Server(encoder, policy, B, L, overlap=overlap)
    return srv.run(lengths, sub["arrival"].astype(np.float64), sub["deadline"].astype(np.float64),
                   token_ids, tok_off, horizon)


def capacity(encoder, dist: str, B: int, L: int, seed: int) -> Tuple[float, float]:
    """(requests per second, seconds per full batch) of one GPU: a full First-Fit batch of
    the length distribution, CUDA-graph replayed."""
    import torch
    import tcb_workload as wl
    from . import tcb_pack
    lengths = wl.lengths_filling(dist, B, L, seed, 0.995)
    plan = tcb_pack(lengths, L, B)
    st = torch.from_numpy(plan.segtab()).cuda()
    ids = torch.zeros(max(int(plan.info["total_tokens"]), 1), dtype=torch.int32, device="cuda")
    rows = encoder.alloc_rows(plan.num_slots)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(2):
            encoder.encoder_forward(plan, st, ids, rows, stream=s)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        encoder.encoder_forward(plan, st, ids, rows, stream=s)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        a.record(s)
        for _ in range(5):
            g.replay()
        b.record(s)
    s.synchronize()
    tau = a.elapsed_time(b) / 5 / 1e3
    return plan.info["num_placed"] / tau, tau
