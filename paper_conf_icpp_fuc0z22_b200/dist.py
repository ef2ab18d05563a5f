"""Data-parallel runtime: one process per GPU, weights broadcast once, rows sharded.

ConcatBatching rows are independent (the mask of Eq. (6), confines attention to
one request, hence to one row), so the path shards over rows / requests with no data-path
collective (north_star).  NCCL is used exactly once per process lifetime: a
broadcast of the flat weight buffers from rank 0 over NVLink.  The per-step work is each
rank's own packed batch; timing uses a barrier and a max-reduction of device-measured times
after the timed region.
"""
from __future__ import annotations

import os
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

_VEC = ("type_emb", "emb_ln_g", "emb_ln_b", "b_qkv", "b_o", "ln1_g", "ln1_b", "b_1", "b_2",
        "ln2_g", "ln2_b")


def env_rank() -> Tuple[int, int, int]:
    """(rank, local_rank, world_size) from the torchrun environment (1 process if absent)."""
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("LOCAL_RANK", 0)),
            int(os.environ.get("WORLD_SIZE", 1)))


def init(backend: str = "nccl"):
    """Initialise torch.distributed when launched under torchrun; returns (rank, world)."""
    import torch
    import torch.distributed as dist
    rank, local, world = env_rank()
    if world > 1 and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if backend == "nccl":
            torch.cuda.set_device(local)
        dist.init_process_group(backend=backend)
    return rank, world


def weight_layout(model, names: Sequence[str]) -> List[Tuple[str, tuple, bool]]:
    """(name, shape, is_matrix) for every canonical tensor, without drawing values."""
    import tcb_workload as wl
    shapes = wl.weight_shapes(model)
    return [(n, shapes[n], n.split(".")[-1] not in _VEC) for n in names]


def broadcast_weights(model, names: Sequence[str], weights: Optional[Dict[str, np.ndarray]],
                      device, src: int = 0) -> list:
    """Materialise the weights on every rank: rank ``src`` uploads its numpy arrays into two
    flat device buffers (model-dtype matrices, fp32 vectors), one NCCL broadcast each, and
    every rank returns per-tensor views in canonical order.  ``weights`` may be None on
    ranks other than ``src``."""
    import torch
    import torch.distributed as dist
    lay = weight_layout(model, names)
    mat_dt = torch.float32 if model.dtype == "fp32" else torch.bfloat16
    # 16-byte aligned offsets so every view satisfies the kernels' alignment
    def offsets(is_mat, esize):
        off, out = 0, {}
        for n, shp, m in lay:
            if m != is_mat:
                continue
            out[n] = off
            off += int(np.prod(shp))
            off = (off + (16 // esize) - 1) // (16 // esize) * (16 // esize)
        return out, off
    moff, mtot = offsets(True, 2 if mat_dt == torch.bfloat16 else 4)
    voff, vtot = offsets(False, 4)
    flat_m = torch.empty(max(mtot, 1), dtype=mat_dt, device=device)
    flat_v = torch.empty(max(vtot, 1), dtype=torch.float32, device=device)
    rank = dist.get_rank() if dist.is_initialized() else 0
    if rank == src:
        for n, shp, m in lay:
            buf, off = (flat_m, moff[n]) if m else (flat_v, voff[n])
            t = torch.from_numpy(np.ascontiguousarray(weights[n]).reshape(-1))
            buf[off:off + t.numel()].copy_(t.to(buf.dtype))
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.broadcast(flat_m, src)
        dist.broadcast(flat_v, src)
    views = []
    for n, shp, m in lay:
        buf, off = (flat_m, moff[n]) if m else (flat_v, voff[n])
        views.append(buf[off:off + int(np.prod(shp))].view(*shp))
    return views


def shard_rows(num_rows: int, rank: int, world: int) -> Tuple[int, int]:
    """Contiguous row range [lo, hi) of ``rank`` when one global batch of ``num_rows`` rows
    is split over ``world`` ranks (balanced to within one row)."""
    base, extra = divmod(num_rows, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def shard_plan_requests(req_row: np.ndarray, rank: int, world: int, num_rows: int) -> np.ndarray:
    """Indices of the requests whose row falls in ``rank``'s row range (global packing on
    one host, rows dealt out per rank); unplaced requests belong to nobody."""
    lo, hi = shard_rows(num_rows, rank, world)
    return np.nonzero((req_row >= lo) & (req_row < hi))[0]


def rank_seed(seed: int, rank: int) -> int:
    """Independent per-rank request stream (weak scaling: fixed work per GPU)."""
    return seed + 1000 * rank
