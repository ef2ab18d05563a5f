"""TEST INFRASTRUCTURE ONLY -- ctypes shim over the float64 CPU oracle (oracle/oracle.c).

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` / ``--impl
reference`` legs may import this package.  It shares no code with the CUDA path
(``paper_conf_icpp_fuc0z22_b200``) and never imports it.  Every function here is
argument marshalling around the C oracle; the arithmetic is in oracle.c, whose header
lists what pins each step (tests/test_oracle_*.py).

Parity status: the paper prints no worked numeric example, so absolute values are pinned
by closed forms, invariants, brute force and torch f64 (P1-P9), not by
numbers from the paper.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Dict, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")

POLICIES = {"first_fit": 0, "next_fit": 1, "first_fit_decreasing": 2, "naive": 3,
            "length_sorted": 4}
PE_VARIANTS = {"sin_paper": 0, "sin_vaswani": 1, "learned": 2}
ACTS = {"gelu": 0, "relu": 1}


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2 -ffp-contract=off -fopenmp, float64)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC",
               "-shared", "-std=c11", "-Wall", "-o", _SO, _SRC, "-lm"]
        subprocess.check_call(cmd, cwd=_HERE)
    return _SO


class _Cfg(ctypes.Structure):
    _fields_ = [("num_layers", ctypes.c_int32), ("d_model", ctypes.c_int32),
                ("num_heads", ctypes.c_int32), ("d_ff", ctypes.c_int32),
                ("act", ctypes.c_int32), ("pe", ctypes.c_int32), ("emb_ln", ctypes.c_int32),
                ("use_type_emb", ctypes.c_int32), ("ln_eps", ctypes.c_double),
                ("emb_ln_eps", ctypes.c_double), ("emb_scale", ctypes.c_double)]


_lib: Optional[ctypes.CDLL] = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.oracle_pe.restype = ctypes.c_double
    return _lib


def set_num_threads(n: int) -> int:
    """OpenMP thread count of the oracle's parallel loops (the libgomp ICV of the calling
    thread; results never depend on it, see oracle.c).  Returns the count now in effect."""
    lib()
    g = ctypes.CDLL("libgomp.so.1")
    g.omp_set_num_threads(ctypes.c_int(int(n)))
    return int(g.omp_get_max_threads())


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.float64))


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def make_cfg(model) -> _Cfg:
    """Build the C config from any object with ModelConfig-like attributes."""
    return _Cfg(model.num_layers, model.d_model, model.num_heads, model.d_ff,
                ACTS[model.act], PE_VARIANTS[model.pe], int(model.emb_ln),
                int(model.use_type_emb), float(model.ln_eps), float(model.emb_ln_eps),
                float(model.emb_scale))


class OracleError(RuntimeError):
    def __init__(self, code: int):
        super().__init__({-1: "invalid argument", -2: "request too long"}.get(code, str(code)))
        self.code = code


def pack(lengths: Sequence[int], row_len: int, max_rows: int = 0,
         policy: str = "first_fit") -> Dict[str, np.ndarray]:
    """o1: assignment of requests to rows (req_row, req_col, num_rows)."""
    lengths = _i32(lengths)
    n = len(lengths)
    req_row = np.zeros(max(n, 1), np.int32)
    req_col = np.zeros(max(n, 1), np.int32)
    rows = ctypes.c_int32(0)
    rc = lib().oracle_pack(_p(lengths), n, row_len, max_rows, POLICIES[policy], _p(req_row),
                           _p(req_col), ctypes.byref(rows))
    if rc != 0:
        raise OracleError(rc)
    return {"req_row": req_row[:n], "req_col": req_col[:n], "num_rows": int(rows.value)}


def pack_slotted(lengths: Sequence[int], row_len: int, slot_len: int = 0,
                 max_rows: int = 0) -> Dict[str, np.ndarray]:
    """o1 slotted (§4.2, Alg. 2, R26): First-Fit of requests into slots of slot_len words
    (0 = the largest length); requests never straddle a slot."""
    lengths = _i32(lengths)
    n = len(lengths)
    req_row = np.zeros(max(n, 1), np.int32)
    req_col = np.zeros(max(n, 1), np.int32)
    rows = ctypes.c_int32(0)
    z = ctypes.c_int32(0)
    rc = lib().oracle_pack_slotted(_p(lengths), n, row_len, max_rows, slot_len, _p(req_row),
                                   _p(req_col), ctypes.byref(rows), ctypes.byref(z))
    if rc != 0:
        raise OracleError(rc)
    return {"req_row": req_row[:n], "req_col": req_col[:n], "num_rows": int(rows.value),
            "slot_len": int(z.value)}


SCHED_POLICIES = {"das": 0, "fcfs": 1, "sjf": 2, "def": 3}


def sched_batch(policy: str, lengths, arrival, deadline, ids, B: int, L: int,
                eta: float = 0.5, q: float = 0.5):
    """f2: one time slot's batch from the waiting set (Alg. 1 / baselines, R27).
    Returns (row, col) per waiting request, -1 = not chosen."""
    lengths = _i32(lengths)
    n = len(lengths)
    arrival = _f64(arrival)
    deadline = _f64(deadline)
    ids = np.ascontiguousarray(np.asarray(ids, dtype=np.int64))
    row = np.zeros(max(n, 1), np.int32)
    col = np.zeros(max(n, 1), np.int32)
    rc = lib().oracle_sched_batch(SCHED_POLICIES[policy], _p(lengths), _p(arrival),
                                  _p(deadline), _p(ids), n, B, L, ctypes.c_double(eta),
                                  ctypes.c_double(q), _p(row), _p(col))
    if rc != 0:
        raise OracleError(rc)
    return row[:n], col[:n]


def sched_simulate(policy: str, lengths, arrival, deadline, B: int, L: int, slot_time: float,
                   num_slots: int, eta: float = 0.5, q: float = 0.5):
    """The online setting of §5.1: time slot t starts at t * slot_time; the
    waiting set N_t holds requests with arrival <= t*slot_time <= deadline not scheduled
    yet (constraint (12)); each slot schedules one batch.  Returns per request
    (slot, row, col) (-1 if never scheduled) and the total utility sum 1/l (Eq. (9))."""
    lengths = _i32(lengths)
    n = len(lengths)
    arrival, deadline = _f64(arrival), _f64(deadline)
    slot = np.full(n, -1, np.int64)
    row = np.full(n, -1, np.int32)
    col = np.full(n, -1, np.int32)
    for t in range(num_slots):
        now = t * slot_time
        wait = [i for i in range(n) if slot[i] < 0 and arrival[i] <= now <= deadline[i]]
        if not wait:
            continue
        w = np.array(wait, np.int64)
        r, c = sched_batch(policy, lengths[w], arrival[w], deadline[w], w, B, L, eta, q)
        for j, i in enumerate(wait):
            if r[j] >= 0:
                slot[i], row[i], col[i] = t, r[j], c[j]
    utility = float(sum(1.0 / lengths[i] for i in range(n) if slot[i] >= 0))
    return {"slot": slot, "row": row, "col": col, "utility": utility}


def layout(lengths, req_row, req_col, num_rows: int, row_len: int,
           qtile: int = 128) -> Dict[str, np.ndarray]:
    """o1 (layout): segment_ids, positions, tok_index, seg_req, seg_start, cu_seqlens,
    qtile_kv for the packed rows."""
    lengths, req_row, req_col = _i32(lengths), _i32(req_row), _i32(req_col)
    n = len(lengths)
    M = num_rows * row_len
    seg_ids = np.zeros(max(M, 1), np.int32)
    pos = np.zeros(max(M, 1), np.int32)
    tok = np.zeros(max(M, 1), np.int32)
    seg_req = np.zeros(max(n, 1), np.int32)
    seg_start = np.zeros(max(n, 1), np.int32)
    cu = np.zeros(n + 1, np.int32)
    nt = (M + qtile - 1) // qtile
    qkv = np.zeros(max(2 * nt, 1), np.int32)
    S = ctypes.c_int32(0)
    rc = lib().oracle_layout(_p(lengths), n, _p(req_row), _p(req_col), num_rows, row_len,
                             qtile, _p(seg_ids), _p(pos), _p(tok), _p(seg_req), _p(seg_start),
                             _p(cu), _p(qkv), ctypes.byref(S))
    if rc != 0:
        raise OracleError(rc)
    s = int(S.value)
    return {"segment_ids": seg_ids[:M], "positions": pos[:M], "tok_index": tok[:M],
            "seg_req": seg_req[:s], "seg_start": seg_start[:s], "cu_seqlens": cu[:s + 1],
            "qtile_kv": qkv[:2 * nt].reshape(nt, 2), "num_segments": s}


def pe(pos: int, dim: int, d_model: int, variant: str = "sin_paper") -> float:
    return float(lib().oracle_pe(int(pos), int(dim), int(d_model), PE_VARIANTS[variant]))


def linear(x, w, b, res=None, act: str = "none") -> np.ndarray:
    x, w, b = _f64(x), _f64(w), _f64(b)
    rows, k = x.shape
    n = w.shape[0]
    y = np.zeros((rows, n), np.float64)
    r = _f64(res) if res is not None else None
    lib().oracle_linear(_p(x), _p(w), _p(b), _p(r) if r is not None else None, rows, n, k,
                        {"none": 0, "gelu": 1, "relu": 2}[act], _p(y))
    return y


def attention(qkv, segment_ids, num_rows: int, row_len: int, d_model: int,
              num_heads: int) -> np.ndarray:
    qkv = _f64(qkv)
    seg = _i32(segment_ids)
    o = np.zeros((num_rows * row_len, d_model), np.float64)
    lib().oracle_attention(_p(qkv), _p(seg), num_rows, row_len, d_model, num_heads, _p(o))
    return o


def layernorm(z, g, b, eps: float) -> np.ndarray:
    z, g, b = _f64(z), _f64(g), _f64(b)
    y = np.zeros_like(z)
    lib().oracle_layernorm(_p(z), _p(g), _p(b), z.shape[0], z.shape[1], ctypes.c_double(eps),
                           _p(y))
    return y


def _weight_ptrs(weights_in_order):
    arrs = [_f64(w) for w in weights_in_order]
    ptrs = (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])
    return arrs, ptrs


def embed(model, weights: Dict[str, np.ndarray], ids, lay) -> np.ndarray:
    cfg = make_cfg(model)
    arrs = [_f64(weights[n]) for n in ("tok_emb", "pos_emb", "type_emb", "emb_ln_g", "emb_ln_b")]
    seg, pos, tok = _i32(lay["segment_ids"]), _i32(lay["positions"]), _i32(lay["tok_index"])
    ids = _i32(ids)
    M = len(seg)
    x = np.zeros((M, model.d_model), np.float64)
    lib().oracle_embed(ctypes.byref(cfg), *[_p(a) for a in arrs], _p(ids), M, _p(seg), _p(pos),
                       _p(tok), _p(x))
    return x


def encoder_rows(model, weights: Dict[str, np.ndarray], names, ids, lay, row_len: int,
                 rows: Optional[Sequence[int]] = None) -> np.ndarray:
    """o2-o7 over packed rows; returns x [len(rows)*row_len, d] (all rows if rows=None).

    Rows never interact (the mask is block-diagonal inside a row, Eq. (6)), so running a
    subset of rows is the same computation restricted to them.
    """
    seg, pos, tok = _i32(lay["segment_ids"]), _i32(lay["positions"]), _i32(lay["tok_index"])
    num_rows = len(seg) // row_len
    if rows is None:
        rows = list(range(num_rows))
    sel = np.concatenate([np.arange(r * row_len, (r + 1) * row_len) for r in rows]) \
        if len(rows) else np.zeros(0, np.int64)
    seg_s, pos_s, tok_s = _i32(seg[sel]), _i32(pos[sel]), _i32(tok[sel])
    cfg = make_cfg(model)
    arrs, ptrs = _weight_ptrs([weights[n] for n in names])
    ids = _i32(ids)
    x = np.zeros((len(sel), model.d_model), np.float64)
    rc = lib().oracle_encoder(ctypes.byref(cfg), ptrs, len(arrs), _p(ids), len(rows), row_len,
                              _p(seg_s), _p(pos_s), _p(tok_s), _p(x))
    if rc != 0:
        raise OracleError(rc)
    return x


def unpack(x, tok_index, total_tokens: int) -> np.ndarray:
    """o8: request-order outputs [total_tokens, d]; tokens of unplaced requests are NaN."""
    x = _f64(x)
    tok = _i32(tok_index)
    out = np.full((total_tokens, x.shape[1]), np.nan, np.float64)
    lib().oracle_unpack(_p(x), len(tok), x.shape[1], _p(tok), _p(out))
    return out


def run(model, weights, names, lengths, ids, row_len: int, max_rows: int = 0,
        policy: str = "first_fit", slot_len: int = 0) -> Dict[str, np.ndarray]:
    """The whole path: pack -> layout -> encoder -> unpack (request order).  policy
    "slotted" packs into slots of slot_len words (§4.2, R26)."""
    if policy == "slotted":
        pk = pack_slotted(lengths, row_len, slot_len, max_rows)
    else:
        pk = pack(lengths, row_len, max_rows, policy)
    lay = layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], row_len)
    x = encoder_rows(model, weights, names, ids, lay, row_len)
    out = unpack(x, lay["tok_index"], int(np.sum(lengths)))
    return {"pack": pk, "layout": lay, "rows": x, "out": out}


# ---------------------------------------------------------------------------------------
# f4: decoder (§4.2.2; readings R30-R33).  Plain definition, one request alone.
# ---------------------------------------------------------------------------------------
def decoder_stack(model, dec_weights: Dict[str, np.ndarray], dec_names, x, mem) -> np.ndarray:
    """S decoder layers over one request's embedded target prefix x [t, d] with its encoder
    output mem [l, d]: causal self-attention, cross-attention, FFN, post-LN each."""
    cfg = make_cfg(model)
    arrs, ptrs = _weight_ptrs([dec_weights[n] for n in dec_names])
    x = _f64(x).copy()
    mem = _f64(mem)
    rc = lib().oracle_decoder_stack(ctypes.byref(cfg), ptrs, len(arrs), x.shape[0], mem.shape[0],
                                    _p(x), _p(mem))
    if rc != 0:
        raise OracleError(rc)
    return x


def decode_greedy(model, weights, names, dec_weights, dec_names, src_ids, t_max: int,
                  bos: int = 1, eos: int = 2, with_logits: bool = False):
    """Greedy decode of one request alone: tokens y_1.. (stops after EOS or t_max) and,
    optionally, the logits of every step [n_out, vocab]."""
    cfg = make_cfg(model)
    ea, ep = _weight_ptrs([weights[n] for n in names])
    da, dp = _weight_ptrs([dec_weights[n] for n in dec_names])
    src = _i32(src_ids)
    toks = np.zeros(t_max, np.int32)
    n = ctypes.c_int32(0)
    lg = np.zeros((t_max, model.vocab), np.float64) if with_logits else None
    rc = lib().oracle_decode_greedy(ctypes.byref(cfg), ep, len(ea), dp, len(da), model.vocab,
                                    _p(src), len(src), t_max, bos, eos, _p(toks), ctypes.byref(n),
                                    _p(lg) if lg is not None else None)
    if rc != 0:
        raise OracleError(rc)
    k = int(n.value)
    return (toks[:k], lg[:k]) if with_logits else toks[:k]
