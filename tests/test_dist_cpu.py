"""Multi-process host logic of the data-parallel runtime (gloo, world size 2, CPU).

The path shards over rows with no data-path collective: the only collective
is the one-time weight broadcast.  These tests run the real runtime functions under
torch.distributed with the gloo backend on 127.0.0.1.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import tcb_workload as wl
from paper_conf_icpp_fuc0z22_b200 import dist as tdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, mkey, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    model = wl.MODELS[mkey]
    names = wl.weight_names(model)
    w = wl.draw_weights(model, 7) if rank == 0 else None
    views = tdist.broadcast_weights(model, names, w, torch.device("cpu"))
    ref = wl.draw_weights(model, 7)
    ok = True
    for (n, shp, is_mat), t in zip(tdist.weight_layout(model, names), views):
        ok &= tuple(t.shape) == tuple(shp)
        ok &= bool(np.array_equal(t.float().numpy(), ref[n].reshape(shp)))
        ok &= t.data_ptr() % 16 == 0
    # timing reduction as bench.py does it: max of times, sum of tokens
    t = torch.tensor([1.0 + rank, 100.0 * (rank + 1)], dtype=torch.float64)
    tmax, tsum = t.clone(), t.clone()
    dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
    dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
    q.put((rank, ok, float(tmax[0]), float(tsum[1])))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("mkey", ["toy", "transformer-base"])
def test_weight_broadcast_gloo_world2(mkey):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, mkey, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    for rank, ok, tmax, tsum in res:
        assert ok, rank
        assert tmax == 2.0 and tsum == 300.0


def test_shard_rows_partition():
    for rows in (1, 7, 256, 1000):
        for world in (1, 2, 3, 8):
            ranges = [tdist.shard_rows(rows, r, world) for r in range(world)]
            assert ranges[0][0] == 0 and ranges[-1][1] == rows
            for (a, b), (c, d) in zip(ranges, ranges[1:]):
                assert b == c
            sizes = [b - a for a, b in ranges]
            assert max(sizes) - min(sizes) <= 1


def test_shard_plan_requests_covers_placed_once():
    import paper_conf_icpp_fuc0z22_b200 as tcb
    lengths = np.minimum(wl.draw_lengths("paracrawl", 500, 3), 128).astype(np.int32)
    plan = tcb.tcb_pack(lengths, 128, 64)
    req_row = plan.arrays()["req_row"]
    seen = np.zeros(len(lengths), np.int32)
    for r in range(4):
        idx = tdist.shard_plan_requests(req_row, r, 4, plan.info["num_rows"])
        seen[idx] += 1
    assert np.array_equal(seen, (req_row >= 0).astype(np.int32))


def test_rank_streams_are_independent():
    a = wl.draw_lengths("wmt", 100, tdist.rank_seed(40, 0))
    b = wl.draw_lengths("wmt", 100, tdist.rank_seed(40, 1))
    assert not np.array_equal(a, b)


# ---- online serving across ranks (serve_dist, BASELINE configs[4]) -------------------------
def _online_worker(rank, world, port, q):
    from paper_conf_icpp_fuc0z22_b200 import serve_dist as sd
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, rate, tau = 40000, 2.0e5, 4e-3
    sub = sd.substream(rank, world, n, rate, "wmt", 256, tau, seed=40)
    # every rank sees the requests the dispatcher sends it; the ranks partition the stream
    ids = torch.from_numpy(sub["id"].astype(np.int64))
    sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(sizes, torch.tensor([len(ids)], dtype=torch.int64))
    pad = torch.full((int(max(s.item() for s in sizes)),), -1, dtype=torch.int64)
    pad[:len(ids)] = ids
    allid = [torch.zeros_like(pad) for _ in range(world)]
    dist.all_gather(allid, pad)
    union = np.concatenate([a.numpy()[a.numpy() >= 0] for a in allid])
    # per-rank counters reduce as the multi-GPU runner does (sums; max of the serving clock)
    fake = {"tokens": 1000.0 * (rank + 1), "scheduled": 10.0, "utility": 0.5, "expired": 1.0,
            "requests": float(len(ids)), "batches": 3.0, "sim_seconds": 0.1 * (rank + 1),
            "batch_ms": 4.0 + rank, "sched_ms": 0.2}
    red = sd.reduce_results(fake, world)
    q.put((rank, union.tolist() if rank == 0 else None, len(ids),
           sub["arrival"].tolist(), sub["length"].tolist(), red))
    dist.barrier()
    dist.destroy_process_group()


def test_online_substreams_gloo_world2():
    """The multi-rank serving runner's feeding logic: each rank's Poisson(lambda / W) share of
    one global stream (independent thinning), the shares partition the stream (every request
    served by exactly one rank), each share's arrival rate is ~lambda / W with exponential
    gaps, and the whole-job counters reduce as sums with the max serving clock."""
    from paper_conf_icpp_fuc0z22_b200 import serve_dist as sd
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_online_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=240) for _ in procs], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    n, rate = 40000, 2.0e5
    union = np.array(res[0][1])
    assert len(union) == n and np.array_equal(np.sort(union), np.arange(n))
    arr_g, len_g, _ = sd.global_stream(n, rate, "wmt", 256, 4e-3, 40)
    for rank, _, cnt, arr, lens, red in res:
        assert abs(cnt / n - 0.5) < 0.02                        # thinning p = 1/W
        gaps = np.diff(np.array(arr))
        # Poisson(lambda / W): mean gap W / lambda, coefficient of variation ~ 1 (exponential)
        assert abs(gaps.mean() * rate / 2 - 1) < 0.05
        assert abs(gaps.std() / gaps.mean() - 1) < 0.05
        assert np.all(np.isin(np.array(lens), len_g))
        assert red["tokens"] == 3000.0 and red["seconds"] == pytest.approx(0.2)
        assert red["max_batch_ms"] == 5.0 and red["requests"] == n
        assert red["tokens_per_s"] == pytest.approx(15000.0)
    # the same seed gives the same global stream on every rank
    assert np.allclose(np.sort(np.concatenate([r[3] for r in res])), arr_g)
