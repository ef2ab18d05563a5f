"""Shared test helpers: run the oracle and the CUDA path on the same seeded inputs and
compare them (tolerances: DESIGN.md §4, reading R21)."""
import numpy as np

import oracle
import tcb_workload as wl

# R21: per-request normwise max relative error  ||g_r - o_r||_inf / ||o_r||_inf
TOL = {"fp32": 1e-4, "bf16": 2e-2}


def per_request_errors(gpu_rows, ref_rows, segment_ids, seg_bounds):
    """gpu_rows/ref_rows: [slots, d] over the same slots; seg_bounds: {seg: (a, b)} slot
    ranges inside these arrays.  Returns {seg: normwise error}."""
    errs = {}
    for s, (a, b) in seg_bounds.items():
        o = ref_rows[a:b]
        g = gpu_rows[a:b]
        errs[s] = float(np.max(np.abs(g - o)) / max(np.max(np.abs(o)), 1e-30))
    return errs


def oracle_selected_rows(model, weights, names, lengths, ids, row_len, rows, max_rows=0,
                         policy="first_fit", slot_len=0):
    if policy == "slotted":
        pk = oracle.pack_slotted(lengths, row_len, slot_len, max_rows)
    else:
        pk = oracle.pack(lengths, row_len, max_rows, policy)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], row_len)
    x = oracle.encoder_rows(model, weights, names, ids, lay, row_len, rows)
    return pk, lay, x


def segments_in_rows(lay, row_len, rows):
    """{segment: (a, b)} in the coordinates of the concatenated selected rows."""
    seg = lay["segment_ids"]
    out = {}
    for i, r in enumerate(rows):
        base = r * row_len
        for j in range(row_len):
            s = int(seg[base + j])
            if s < 0:
                continue
            a, b = out.get(s, (i * row_len + j, i * row_len + j))
            out[s] = (min(a, i * row_len + j), max(b, i * row_len + j + 1))
    return out


def small_model(name="t", d=64, h=2, f=256, layers=2, dtype="fp32", act="gelu",
                pe="sin_paper", emb_ln=False, vocab=128, max_pos=512):
    return wl.ModelConfig(name, layers, d, h, f, vocab, max_pos, dtype, act, pe, emb_ln, emb_ln,
                          1e-12 if emb_ln else 1e-5, 1e-12 if emb_ln else 1e-5, 1.0)
