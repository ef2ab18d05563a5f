"""ctypes binding of libtcb.so (include/tcb.h, include/tcb_ops.h): argument marshalling only.

Every step of the path runs in the library's CUDA kernels.  Loading fails loudly when the
library is missing; device calls without a B200 return TCB_ERR_NO_DEVICE (there is no CPU
fallback anywhere in this package).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.path.join(_HERE, "libtcb.so")

TCB_OK = 0
STATUS = {0: "TCB_OK", -1: "TCB_ERR_INVALID_ARGUMENT", -2: "TCB_ERR_REQUEST_TOO_LONG",
          -3: "TCB_ERR_UNSUPPORTED", -4: "TCB_ERR_CUDA", -5: "TCB_ERR_OUT_OF_MEMORY",
          -6: "TCB_ERR_WORKSPACE_TOO_SMALL", -7: "TCB_ERR_NO_DEVICE"}
POLICIES = {"first_fit": 0, "next_fit": 1, "first_fit_decreasing": 2, "naive": 3,
            "length_sorted": 4}
EPILOGUES = {"bias": 0, "bias_gelu": 1, "bias_relu": 2, "bias_residual": 3}
KCLASSES = ["embed", "gemm_qkv", "attention", "gemm_o", "layernorm", "gemm_ffn1", "gemm_ffn2",
            "unpack"]

# Every symbol include/tcb.h and include/tcb_ops.h declare (checked by the CPU tests).
EXPORTS = ["tcb_last_error", "tcb_version", "tcb_pack", "tcb_pack_slotted", "tcb_plan_destroy",
           "tcb_plan_info_get", "tcb_plan_copy", "tcb_plan_segtab_words",
           "tcb_plan_write_segtab", "tcb_weights_count", "tcb_weights_create",
           "tcb_weights_destroy", "tcb_workspace_size", "tcb_embed", "tcb_encoder_forward",
           "tcb_encoder_forward_unpacked",
           "tcb_unpack", "tcb_session_create", "tcb_session_run", "tcb_session_wait",
           "tcb_session_destroy", "tcb_launch_count", "tcb_profile_enable", "tcb_profile_collect", "tcb_profile_snapshot",
           "tcb_op_linear", "tcb_op_linear_ln", "tcb_op_attention", "tcb_op_layernorm",
           "tcb_sched_batch", "tcb_sched_create", "tcb_sched_destroy", "tcb_sched_submit",
           "tcb_sched_next_batch", "tcb_sched_stats_get",
           "tcb_decoder_weights_count", "tcb_decoder_create", "tcb_decoder_destroy",
           "tcb_decode_greedy", "tcb_decoder_stats", "tcb_decoder_last_logits"]
SCHED_POLICIES = {"das": 0, "fcfs": 1, "sjf": 2, "def": 3}


class TcbError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class PlanInfo(ctypes.Structure):
    _fields_ = [("num_requests", ctypes.c_int32), ("num_placed", ctypes.c_int32),
                ("num_rows", ctypes.c_int32), ("row_len", ctypes.c_int32),
                ("num_segments", ctypes.c_int32), ("slot_len", ctypes.c_int32),
                ("total_tokens", ctypes.c_int64), ("placed_tokens", ctypes.c_int64),
                ("num_slots", ctypes.c_int64), ("qtiles", ctypes.c_int64),
                ("kv_tiles_visited", ctypes.c_int64), ("kv_tiles_dense", ctypes.c_int64),
                ("useful_score_elems", ctypes.c_int64),
                ("executed_score_elems", ctypes.c_int64),
                ("softmax_score_elems", ctypes.c_int64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class SchedStats(ctypes.Structure):
    _fields_ = [("submitted", ctypes.c_int64), ("waiting", ctypes.c_int64),
                ("scheduled", ctypes.c_int64), ("expired", ctypes.c_int64),
                ("batches", ctypes.c_int64), ("utility", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class DecodeStats(ctypes.Structure):
    _fields_ = [("steps", ctypes.c_int32), ("rows_computed", ctypes.c_int64),
                ("tokens_generated", ctypes.c_int64), ("kv_bytes_peak", ctypes.c_int64),
                ("kv_bytes_avg", ctypes.c_double), ("ms_total", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class ModelConfig(ctypes.Structure):
    _fields_ = [("num_layers", ctypes.c_int32), ("d_model", ctypes.c_int32),
                ("num_heads", ctypes.c_int32), ("d_ff", ctypes.c_int32),
                ("vocab", ctypes.c_int32), ("max_pos", ctypes.c_int32),
                ("dtype", ctypes.c_int32), ("act", ctypes.c_int32), ("pe", ctypes.c_int32),
                ("emb_ln", ctypes.c_int32), ("use_type_emb", ctypes.c_int32),
                ("ln_eps", ctypes.c_float), ("emb_ln_eps", ctypes.c_float),
                ("emb_scale", ctypes.c_float)]


_lib = None
P = ctypes.c_void_p
I32 = ctypes.c_int32
I64 = ctypes.c_int64


def lib() -> ctypes.CDLL:
    """Load libtcb.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO_PATH):
        raise ImportError(f"{SO_PATH} is missing: run __graft_entry__.build() "
                          "(python -c 'import __graft_entry__ as g; g.build()')")
    L = ctypes.CDLL(SO_PATH)
    sig = {
        "tcb_last_error": (ctypes.c_char_p, []),
        "tcb_version": (ctypes.c_char_p, []),
        "tcb_pack": (I32, [P, I32, I32, I32, I32, ctypes.POINTER(P)]),
        "tcb_pack_slotted": (I32, [P, I32, I32, I32, I32, ctypes.POINTER(P)]),
        "tcb_plan_destroy": (None, [P]),
        "tcb_plan_info_get": (I32, [P, ctypes.POINTER(PlanInfo)]),
        "tcb_plan_copy": (I32, [P] + [P] * 8),
        "tcb_plan_segtab_words": (I64, [P]),
        "tcb_plan_write_segtab": (I32, [P, P, I64]),
        "tcb_weights_count": (I32, [ctypes.POINTER(ModelConfig)]),
        "tcb_weights_create": (I32, [ctypes.POINTER(ModelConfig), P, I32, ctypes.POINTER(P)]),
        "tcb_weights_destroy": (None, [P]),
        "tcb_workspace_size": (I32, [ctypes.POINTER(ModelConfig), I64,
                                     ctypes.POINTER(ctypes.c_size_t)]),
        "tcb_embed": (I32, [P, P, P, P, P, P, P, P]),
        "tcb_encoder_forward": (I32, [P, P, P, P, P, P, ctypes.c_size_t, P]),
        "tcb_encoder_forward_unpacked": (I32, [P, P, P, P, P, P, P, ctypes.c_size_t, P]),
        "tcb_unpack": (I32, [P, P, P, P, P, P]),
        "tcb_session_create": (I32, [P, I32, I32, I64, ctypes.POINTER(P)]),
        "tcb_session_run": (I32, [P, P, P, P, P, P, ctypes.POINTER(I64)]),
        "tcb_session_wait": (I32, [P, I64]),
        "tcb_session_destroy": (None, [P]),
        "tcb_launch_count": (I64, []),
        "tcb_profile_enable": (I32, [I32]),
        "tcb_profile_collect": (I32, [P, P]),
        "tcb_profile_snapshot": (I32, [P, P]),
        "tcb_op_linear": (I32, [I32, I64, I32, I32, P, P, P, P, I32, P, P]),
        "tcb_op_linear_ln": (I32, [I64, I32, I32, P, P, P, P, P, P, ctypes.c_float, P, P, P]),
        "tcb_op_attention": (I32, [I32, I64, I32, I32, P, P, P, P, P]),
        "tcb_op_layernorm": (I32, [I32, I64, I32, P, P, P, ctypes.c_float, P, P, P]),
        "tcb_sched_batch": (I32, [I32, P, P, P, P, I32, I32, I32, ctypes.c_double,
                                  ctypes.c_double, P, P]),
        "tcb_sched_create": (I32, [I32, I32, I32, ctypes.c_double, ctypes.c_double,
                                   ctypes.POINTER(P)]),
        "tcb_sched_destroy": (None, [P]),
        "tcb_sched_submit": (I32, [P, I32, P, P, P, P]),
        "tcb_sched_next_batch": (I32, [P, ctypes.c_double, P, P, I32, ctypes.POINTER(I32),
                                       ctypes.POINTER(P)]),
        "tcb_sched_stats_get": (I32, [P, ctypes.POINTER(SchedStats)]),
        "tcb_decoder_weights_count": (I32, [ctypes.POINTER(ModelConfig)]),
        "tcb_decoder_create": (I32, [P, P, I32, I32, I64, I32, ctypes.POINTER(P)]),
        "tcb_decoder_destroy": (None, [P]),
        "tcb_decode_greedy": (I32, [P, P, P, I32, P, P, P]),
        "tcb_decoder_stats": (I32, [P, ctypes.POINTER(DecodeStats)]),
        "tcb_decoder_last_logits": (I32, [P, P, I64, ctypes.POINTER(I32)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L


def check(status: int) -> None:
    if status != TCB_OK:
        raise TcbError(status, lib().tcb_last_error().decode())
