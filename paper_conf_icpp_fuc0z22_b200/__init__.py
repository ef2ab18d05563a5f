"""B200-native ConcatBatching encoder (TCB, Fu et al., ICPP'22) -- Python binding.

Thin layer over libtcb.so (include/tcb.h): PyTorch supplies device memory and streams;
every step of the path (pack_embed, tcgen05 GEMMs, segment-masked attention, LayerNorm,
unpack) runs in the library's sm_100a kernels.  Names follow the C ABI:

    plan = tcb_pack(lengths, row_len, max_rows, policy)          # host, C++
    enc  = Encoder(model_cfg, weights)                           # device weights
    rows = enc.encoder_forward(plan, d_segtab, d_token_ids)      # [B*L, d] on the GPU
    out  = enc.unpack(plan, d_segtab, rows)                      # [total_tokens, d]
"""
from __future__ import annotations

import ctypes
from typing import Dict, Optional, Sequence

import numpy as np

from . import _lib
from ._lib import KCLASSES, POLICIES, TcbError, check, lib

__all__ = ["Plan", "Encoder", "Decoder", "Scheduler", "sched_batch", "tcb_pack", "tcb_pack_slotted", "op_linear", "op_linear_ln", "op_attention", "op_layernorm",
           "launch_count", "profile_enable", "profile_collect", "profile_snapshot", "TcbError",
           "KCLASSES", "Session"]

_DTYPES = {"fp32": 0, "bf16": 1}
_ACTS = {"gelu": 0, "relu": 1}
_PES = {"sin_paper": 0, "sin_vaswani": 1, "learned": 2}
_VEC_WEIGHTS = ("type_emb", "emb_ln_g", "emb_ln_b", "b_qkv", "b_o", "ln1_g", "ln1_b", "b_1",
                "b_2", "ln2_g", "ln2_b")


def _ptr(a) -> ctypes.c_void_p:
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data_as(ctypes.c_void_p)
    return ctypes.c_void_p(a.data_ptr())  # torch tensor


def _stream_ptr(stream) -> ctypes.c_void_p:
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


class Plan:
    """A packed batch (host): row assignment + segment table.  Wraps tcb_plan*."""

    def __init__(self, handle: ctypes.c_void_p):
        self._h = handle
        info = _lib.PlanInfo()
        check(lib().tcb_plan_info_get(self._h, ctypes.byref(info)))
        self.info = info.as_dict()

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        try:
            if h and _lib._lib is not None:
                _lib._lib.tcb_plan_destroy(h)
        except Exception:  # interpreter shutdown
            pass

    @property
    def handle(self):
        return self._h

    @property
    def num_slots(self) -> int:
        return self.info["num_slots"]

    def arrays(self) -> Dict[str, np.ndarray]:
        i = self.info
        n, S, M, Q = i["num_requests"], i["num_segments"], i["num_slots"], i["qtiles"]
        out = {"req_row": np.zeros(max(n, 1), np.int32), "req_col": np.zeros(max(n, 1), np.int32),
               "seg_req": np.zeros(max(S, 1), np.int32), "seg_start": np.zeros(max(S, 1), np.int32),
               "cu_seqlens": np.zeros(S + 1, np.int32),
               "segment_ids": np.zeros(max(M, 1), np.int32),
               "positions": np.zeros(max(M, 1), np.int32),
               "qtile_kv": np.zeros(max(2 * Q, 1), np.int32)}
        check(lib().tcb_plan_copy(self._h, *[_ptr(out[k]) for k in (
            "req_row", "req_col", "seg_req", "seg_start", "cu_seqlens", "segment_ids",
            "positions", "qtile_kv")]))
        out["req_row"], out["req_col"] = out["req_row"][:n], out["req_col"][:n]
        out["seg_req"], out["seg_start"] = out["seg_req"][:S], out["seg_start"][:S]
        out["segment_ids"], out["positions"] = out["segment_ids"][:M], out["positions"][:M]
        out["qtile_kv"] = out["qtile_kv"][:2 * Q].reshape(Q, 2)
        return out

    def segtab(self) -> np.ndarray:
        """The device form of the plan (int32 words; copy it to the GPU as-is)."""
        words = int(lib().tcb_plan_segtab_words(self._h))
        buf = np.zeros(words, np.int32)
        check(lib().tcb_plan_write_segtab(self._h, _ptr(buf), words))
        return buf


def tcb_pack(lengths: Sequence[int], row_len: int, max_rows: int = 0,
             policy: str = "first_fit") -> Plan:
    """Assign requests to rows (C++ packer).  See include/tcb.h tcb_pack."""
    arr = np.ascontiguousarray(np.asarray(lengths, dtype=np.int32))
    h = ctypes.c_void_p()
    check(lib().tcb_pack(_ptr(arr) if len(arr) else None, len(arr), int(row_len),
                         int(max_rows), POLICIES[policy], ctypes.byref(h)))
    return Plan(h)


def tcb_pack_slotted(lengths: Sequence[int], row_len: int, slot_len: int = 0,
                     max_rows: int = 0) -> Plan:
    """Slotted ConcatBatching (C++ packer): First-Fit into slots of slot_len words
    (0 = the largest length).  See include/tcb.h tcb_pack_slotted."""
    arr = np.ascontiguousarray(np.asarray(lengths, dtype=np.int32))
    h = ctypes.c_void_p()
    check(lib().tcb_pack_slotted(_ptr(arr) if len(arr) else None, len(arr), int(row_len),
                                 int(max_rows), int(slot_len), ctypes.byref(h)))
    return Plan(h)


def sched_batch(policy: str, lengths, arrival, deadline, ids, B: int, L: int,
                eta: float = 0.5, q: float = 0.5):
    """One time slot's batch from a waiting set (C++ scheduler, include/tcb.h §5).
    Returns (row, col) per request (-1 = not in the batch)."""
    lengths = np.ascontiguousarray(np.asarray(lengths, dtype=np.int32))
    n = len(lengths)
    arrival = np.ascontiguousarray(np.asarray(arrival, dtype=np.float64))
    deadline = np.ascontiguousarray(np.asarray(deadline, dtype=np.float64))
    ids = np.ascontiguousarray(np.asarray(ids, dtype=np.int64))
    row = np.zeros(max(n, 1), np.int32)
    col = np.zeros(max(n, 1), np.int32)
    check(lib().tcb_sched_batch(_lib.SCHED_POLICIES[policy], _ptr(lengths), _ptr(arrival),
                                _ptr(deadline), _ptr(ids), n, int(B), int(L), float(eta),
                                float(q), _ptr(row), _ptr(col)))
    return row[:n], col[:n]


class Scheduler:
    """Online request scheduler (DAS / FCFS / SJF / DEF) over B x L batches; wraps
    tcb_scheduler*.  next_batch(now) returns (ids, lengths, Plan of exactly B rows)."""

    def __init__(self, policy: str, batch_rows: int, row_len: int, eta: float = 0.5,
                 q: float = 0.5):
        h = ctypes.c_void_p()
        check(lib().tcb_sched_create(_lib.SCHED_POLICIES[policy], int(batch_rows),
                                     int(row_len), float(eta), float(q), ctypes.byref(h)))
        self._h = h
        self.B, self.L = int(batch_rows), int(row_len)
        self._cap = 1024

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        try:
            if h and _lib._lib is not None:
                _lib._lib.tcb_sched_destroy(h)
        except Exception:  # interpreter shutdown
            pass

    def submit(self, ids, lengths, arrival, deadline) -> None:
        ids = np.ascontiguousarray(np.asarray(ids, dtype=np.int64))
        lengths = np.ascontiguousarray(np.asarray(lengths, dtype=np.int32))
        arrival = np.ascontiguousarray(np.asarray(arrival, dtype=np.float64))
        deadline = np.ascontiguousarray(np.asarray(deadline, dtype=np.float64))
        check(lib().tcb_sched_submit(self._h, len(ids), _ptr(ids), _ptr(lengths),
                                     _ptr(arrival), _ptr(deadline)))

    def next_batch(self, now: float, with_plan: bool = True):
        cap = max(self._cap, self.B * self.L)          # a batch holds at most B*L requests
        ids = np.zeros(cap, np.int64)
        lens = np.zeros(cap, np.int32)
        n = ctypes.c_int32(0)
        h = ctypes.c_void_p()
        check(lib().tcb_sched_next_batch(self._h, float(now), _ptr(ids), _ptr(lens), cap,
                                         ctypes.byref(n), ctypes.byref(h) if with_plan else None))
        k = int(n.value)
        return ids[:k], lens[:k], (Plan(h) if with_plan else None)

    def stats(self) -> Dict[str, float]:
        st = _lib.SchedStats()
        check(lib().tcb_sched_stats_get(self._h, ctypes.byref(st)))
        return st.as_dict()


def launch_count() -> int:
    return int(lib().tcb_launch_count())


def profile_enable(on: bool) -> None:
    check(lib().tcb_profile_enable(1 if on else 0))


def profile_collect() -> Dict[str, tuple]:
    ms = np.zeros(len(KCLASSES), np.float64)
    n = np.zeros(len(KCLASSES), np.int64)
    check(lib().tcb_profile_collect(_ptr(ms), _ptr(n)))
    return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(KCLASSES)}


def profile_snapshot() -> Dict[str, tuple]:
    """Per-class (ms, launches) of the current records without clearing them (the records of
    a graph captured with profiling on are re-timed by every replay)."""
    ms = np.zeros(len(KCLASSES), np.float64)
    n = np.zeros(len(KCLASSES), np.int64)
    check(lib().tcb_profile_snapshot(_ptr(ms), _ptr(n)))
    return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(KCLASSES)}


class Encoder:
    """Device weights + workspace for one model config; runs the C-ABI device calls.

    ``model`` is any object with tcb_workload.ModelConfig attributes; ``weights`` maps the
    canonical names (tcb_workload.weight_names) to fp32 numpy arrays (already rounded to
    bf16 values for bf16 models).  Matrices are uploaded in the model dtype, vectors fp32.
    """

    def __init__(self, model, weights: Dict[str, np.ndarray], names: Sequence[str],
                 device: str = "cuda", tensors: Optional[list] = None):
        import torch
        self.model = model
        self.device = torch.device(device)
        self.dtype = torch.float32 if model.dtype == "fp32" else torch.bfloat16
        self.cfg = _lib.ModelConfig(model.num_layers, model.d_model, model.num_heads,
                                    model.d_ff, model.vocab, model.max_pos, _DTYPES[model.dtype],
                                    _ACTS[model.act], _PES[model.pe], int(model.emb_ln),
                                    int(model.use_type_emb), model.ln_eps, model.emb_ln_eps,
                                    model.emb_scale)
        if tensors is None:
            tensors = []
            for n in names:
                base = n.split(".")[-1]
                dt = torch.float32 if base in _VEC_WEIGHTS else self.dtype
                tensors.append(torch.from_numpy(np.ascontiguousarray(weights[n]))
                               .to(device=self.device, dtype=dt).contiguous())
        self.tensors = tensors
        ptrs = (ctypes.c_void_p * len(tensors))(*[t.data_ptr() for t in tensors])
        h = ctypes.c_void_p()
        check(lib().tcb_weights_create(ctypes.byref(self.cfg), ptrs, len(tensors),
                                       ctypes.byref(h)))
        self._h = h
        self._ws = None

    @staticmethod
    def weight_dtypes(model, names):
        """(name, is_matrix) for each canonical tensor (used by the broadcast runtime)."""
        return [(n, n.split(".")[-1] not in _VEC_WEIGHTS) for n in names]

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        try:
            if h and _lib._lib is not None:
                _lib._lib.tcb_weights_destroy(h)
        except Exception:  # interpreter shutdown
            pass

    def workspace_bytes(self, num_slots: int) -> int:
        b = ctypes.c_size_t(0)
        check(lib().tcb_workspace_size(ctypes.byref(self.cfg), int(num_slots), ctypes.byref(b)))
        return int(b.value)

    def workspace(self, num_slots: int):
        import torch
        need = self.workspace_bytes(num_slots)
        if self._ws is None or self._ws.numel() < need:
            self._ws = torch.empty(need, dtype=torch.uint8, device=self.device)
        return self._ws

    def alloc_rows(self, num_slots: int):
        import torch
        return torch.empty((num_slots, self.model.d_model), dtype=self.dtype, device=self.device)

    def embed(self, plan: Plan, d_segtab, d_ids, rows, d_seg=None, d_pos=None, stream=None):
        check(lib().tcb_embed(self._h, plan.handle, _ptr(d_segtab), _ptr(d_ids), _ptr(rows),
                              _ptr(d_seg), _ptr(d_pos), _stream_ptr(stream)))
        return rows

    def encoder_forward(self, plan: Plan, d_segtab, d_ids, rows=None, stream=None):
        M = plan.num_slots
        if rows is None:
            rows = self.alloc_rows(M)
        ws = self.workspace(M)
        check(lib().tcb_encoder_forward(self._h, plan.handle, _ptr(d_segtab), _ptr(d_ids),
                                        _ptr(rows), _ptr(ws), ws.numel(), _stream_ptr(stream)))
        return rows

    def encoder_forward_unpacked(self, plan: Plan, d_segtab, d_ids, out=None, rows=None,
                                 stream=None):
        """tcb_encoder_forward + tcb_unpack in one call (the unpack fused into the last
        FFN2 + LN2 where possible); returns out [total_tokens, d_model]."""
        import torch
        M = plan.num_slots
        if rows is None:
            rows = self.alloc_rows(M)
        if out is None:
            out = torch.zeros((plan.info["total_tokens"], self.model.d_model), dtype=self.dtype,
                              device=self.device)
        ws = self.workspace(M)
        check(lib().tcb_encoder_forward_unpacked(self._h, plan.handle, _ptr(d_segtab), _ptr(d_ids),
                                                 _ptr(rows), _ptr(out), _ptr(ws), ws.numel(),
                                                 _stream_ptr(stream)))
        return out

    def unpack(self, plan: Plan, d_segtab, rows, out=None, stream=None):
        import torch
        if out is None:
            out = torch.zeros((plan.info["total_tokens"], self.model.d_model), dtype=self.dtype,
                              device=self.device)
        check(lib().tcb_unpack(self._h, plan.handle, _ptr(d_segtab), _ptr(rows), _ptr(out),
                               _stream_ptr(stream)))
        return out

    def session(self, num_rows: int, row_len: int, max_tokens: int) -> "Session":
        """Host-buffer path (tcb_session_*): device buffers for a fixed B x L shape, owned by
        the library; each run takes a host plan, host token ids and a host output buffer."""
        return Session(self, num_rows, row_len, max_tokens)

    def run(self, lengths, token_ids, row_len: int, max_rows: int = 0,
            policy: str = "first_fit", slot_len: int = 0):
        """Host arrays in, device outputs out: pack -> H2D -> forward -> unpack.
        policy "slotted" packs with tcb_pack_slotted(slot_len)."""
        import torch
        if policy == "slotted":
            plan = tcb_pack_slotted(lengths, row_len, slot_len, max_rows)
        else:
            plan = tcb_pack(lengths, row_len, max_rows, policy)
        d_segtab = torch.from_numpy(plan.segtab()).to(self.device)
        d_ids = torch.from_numpy(np.ascontiguousarray(token_ids, dtype=np.int32)).to(self.device)
        rows = self.encoder_forward(plan, d_segtab, d_ids)
        out = self.unpack(plan, d_segtab, rows)
        return plan, rows, out


class Session:
    """tcb_session_*: host buffers in, host buffers out, two slots in turn (include/tcb.h)."""

    def __init__(self, enc: Encoder, num_rows: int, row_len: int, max_tokens: int):
        self.enc = enc
        h = ctypes.c_void_p()
        check(lib().tcb_session_create(enc._h, int(num_rows), int(row_len), int(max_tokens),
                                       ctypes.byref(h)))
        self._h = h

    def run(self, plan: Plan, h_ids, h_out, stream=None, copy_stream=None) -> int:
        """Enqueue one batch: h_ids (host int32 tensor / array, pinned for async copies) ->
        h_out (host tensor [>= total_tokens, d_model], model dtype).  Returns the ticket."""
        t = ctypes.c_int64(-1)
        cs = ctypes.c_void_p(copy_stream.cuda_stream) if copy_stream is not None else ctypes.c_void_p()
        check(lib().tcb_session_run(self._h, plan.handle, _ptr(h_ids), _ptr(h_out),
                                    _stream_ptr(stream), cs, ctypes.byref(t)))
        return int(t.value)

    def wait(self, ticket: int) -> None:
        check(lib().tcb_session_wait(self._h, int(ticket)))

    def __del__(self):
        try:
            if getattr(self, "_h", None):
                lib().tcb_session_destroy(self._h)
                self._h = None
        except Exception:
            pass


def op_linear(A, W, bias, R=None, epilogue: str = "bias", out=None, stream=None):
    import torch
    M, K = A.shape
    N = W.shape[0]
    if out is None:
        out = torch.empty((M, N), dtype=A.dtype, device=A.device)
    dt = 0 if A.dtype == torch.float32 else 1
    check(lib().tcb_op_linear(dt, M, N, K, _ptr(A), _ptr(W), _ptr(bias), _ptr(R),
                              _lib.EPILOGUES[epilogue], _ptr(out), _stream_ptr(stream)))
    return out


def op_linear_ln(A, W, bias, R, gamma, beta, eps: float, seg_ids=None, out=None, stream=None):
    """C = LayerNorm(A W^T + bias + R) * gamma + beta (bf16, N == 512), one fused kernel."""
    import torch
    M, K = A.shape
    N = W.shape[0]
    if out is None:
        out = torch.empty((M, N), dtype=A.dtype, device=A.device)
    check(lib().tcb_op_linear_ln(M, N, K, _ptr(A), _ptr(W), _ptr(bias), _ptr(R), _ptr(gamma),
                                 _ptr(beta), float(eps), _ptr(seg_ids), _ptr(out),
                                 _stream_ptr(stream)))
    return out


def op_attention(qkv, seg_ids, d_segtab, num_heads: int, out=None, stream=None):
    import torch
    M, three_d = qkv.shape
    d = three_d // 3
    if out is None:
        out = torch.empty((M, d), dtype=qkv.dtype, device=qkv.device)
    dt = 0 if qkv.dtype == torch.float32 else 1
    check(lib().tcb_op_attention(dt, M, d, num_heads, _ptr(qkv), _ptr(seg_ids), _ptr(d_segtab),
                                 _ptr(out), _stream_ptr(stream)))
    return out


def op_layernorm(Z, g, b, eps: float, seg_ids=None, out=None, stream=None):
    import torch
    rows, d = Z.shape
    if out is None:
        out = torch.empty_like(Z)
    dt = 0 if Z.dtype == torch.float32 else 1
    check(lib().tcb_op_layernorm(dt, rows, d, _ptr(Z), _ptr(g), _ptr(b), float(eps),
                                 _ptr(seg_ids), _ptr(out), _stream_ptr(stream)))
    return out


class Decoder:
    """Greedy auto-regressive decoder of the Seq2Seq setting (include/tcb_decoder.h, f4) over
    an Encoder's weights: tied E_tok, causal self-attention with a KV cache per request,
    cross-attention over the request's own segment of the packed encoder rows, early memory
    cleaning (finished requests leave the active set).  Argument marshalling only."""

    def __init__(self, encoder: "Encoder", dec_weights: Dict[str, np.ndarray],
                 dec_names: Sequence[str], max_requests: int, max_slots: int, max_target: int):
        import torch
        self.encoder = encoder
        self.max_target = int(max_target)
        dev = encoder.device
        self.tensors = []
        for n in dec_names:
            base = n.split(".")[-1]
            dt = torch.float32 if (base.startswith("b_") or base.startswith("ln")) else encoder.dtype
            self.tensors.append(torch.from_numpy(np.ascontiguousarray(dec_weights[n]))
                                .to(device=dev, dtype=dt).contiguous())
        ptrs = (ctypes.c_void_p * len(self.tensors))(*[t.data_ptr() for t in self.tensors])
        h = ctypes.c_void_p()
        check(lib().tcb_decoder_create(encoder._h, ptrs, len(self.tensors), int(max_requests),
                                       int(max_slots), int(max_target), ctypes.byref(h)))
        self._h = h

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        try:
            if h and _lib._lib is not None:
                _lib._lib.tcb_decoder_destroy(h)
        except Exception:  # interpreter shutdown
            pass

    def decode(self, plan: "Plan", enc_rows, early_clean: bool = True, tokens=None, stream=None):
        """Returns (device tokens [n, max_target] int32 with -1 past the end, host lengths)."""
        import torch
        n = plan.info["num_requests"]
        if tokens is None:
            tokens = torch.empty((max(n, 1), self.max_target), dtype=torch.int32,
                                 device=self.encoder.device)
        lens = np.zeros(max(n, 1), np.int32)
        check(lib().tcb_decode_greedy(self._h, plan.handle, _ptr(enc_rows), int(bool(early_clean)),
                                      _ptr(tokens), lens.ctypes.data_as(ctypes.c_void_p),
                                      _stream_ptr(stream)))
        return tokens, lens[:n]

    def stats(self) -> Dict[str, float]:
        st = _lib.DecodeStats()
        check(lib().tcb_decoder_stats(self._h, ctypes.byref(st)))
        return st.as_dict()

    def last_logits(self) -> np.ndarray:
        """bf16 logits of the last step as float32 [rows, vocab]."""
        import torch
        V = self.encoder.model.vocab
        cap = self.encoder.model.vocab * max(1, 4096)
        buf = torch.empty(cap, dtype=torch.bfloat16)
        rows = ctypes.c_int32(0)
        check(lib().tcb_decoder_last_logits(self._h, ctypes.c_void_p(buf.data_ptr()), cap,
                                            ctypes.byref(rows)))
        return buf[:rows.value * V].float().numpy().reshape(rows.value, V)
