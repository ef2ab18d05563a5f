"""Pins P4 / P7 / P9 -- the method's correctness claim, checked on the oracle itself.

PAPER.md:500-506 (§3): default inference on concatenated requests "would generate wrong
results", so TCB customises PE (§4.1.1) and self-attention (§4.1.2, Eq. (5)-(6)) "to
guarantee inference correctness"; only the diagonal blocks Q_i K_i^T are useful
(PAPER.md:686-697).  Hence: each request's output inside a concatenated row equals that
request run alone, whatever the packing.  In the f64 oracle (fixed-order sums; masked
terms add exact zeros) this holds BITWISE.
"""
import itertools

import numpy as np
import pytest

import oracle
import tcb_workload as wl


def _toy(seed=2, pe="sin_paper", act="gelu", emb_ln=False):
    cfg = wl.ModelConfig("t", 2, 64, 2, 256, 128, 64, "fp32", act, pe, emb_ln, emb_ln,
                         1e-5, 1e-5, 1.0)
    return cfg, wl.draw_weights(cfg, seed), wl.weight_names(wl.ModelConfig(
        "t", 2, 64, 2, 256, 128, 64, "fp32", act, pe, emb_ln, emb_ln, 1e-5, 1e-5, 1.0))


def _alone(cfg, w, names, ids, length):
    """One request alone, one row of exactly its length, no padding."""
    pk = oracle.pack([length], length)
    lay = oracle.layout([length], pk["req_row"], pk["req_col"], 1, length)
    return oracle.encoder_rows(cfg, w, names, ids, lay, length)


@pytest.mark.parametrize("pe,emb_ln", [("sin_paper", False), ("sin_vaswani", False),
                                       ("learned", True)])
def test_concat_equals_alone_bitwise(pe, emb_ln):
    cfg, w, names = _toy(pe=pe, emb_ln=emb_ln)
    lengths = wl.draw_lengths("uniform_3_16", 8, 0)          # C1: [14,11,10,6,7,3,4,3]
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 1)
    res = oracle.run(cfg, w, names, lengths, ids, 32)
    cu = np.concatenate([[0], np.cumsum(lengths)])
    for r, l in enumerate(lengths):
        alone = _alone(cfg, w, names, ids[cu[r]:cu[r + 1]], int(l))
        assert np.array_equal(res["out"][cu[r]:cu[r + 1]], alone), r


def test_concat_independent_of_offset_row_and_policy_bitwise():
    """(b) any column offset, (c) any row, P7: FF / NF / FFD / Naive / Sorted agree."""
    cfg, w, names = _toy(seed=4)
    rng = np.random.default_rng(12)
    lengths = rng.integers(2, 20, size=13).astype(np.int32)
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 5)
    outs = {}
    for pol in oracle.POLICIES:
        L = 40 if pol not in ("naive", "length_sorted") else int(-(-lengths.max() // 8) * 8)
        outs[pol] = oracle.run(cfg, w, names, lengths, ids, L, 0, pol)["out"]
    ref = outs["first_fit"]
    assert not np.isnan(ref).any()
    for pol, o in outs.items():
        assert np.array_equal(o, ref), pol
    # the same stream packed into longer rows
    o64 = oracle.run(cfg, w, names, lengths, ids, 64)["out"]
    assert np.array_equal(o64, ref)


def test_every_valid_packing_of_a_tiny_input_bitwise():
    """(d) enumerate all set partitions x within-row orders of 4 requests into rows of 12."""
    cfg, w, names = _toy(seed=6)
    lengths = np.array([5, 3, 4, 2], np.int32)
    L = 12
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 8)
    ref = oracle.run(cfg, w, names, lengths, ids, L)["out"]
    n = len(lengths)
    cnt = 0
    for assign in itertools.product(range(n), repeat=n):
        rows = {}
        for r, k in enumerate(assign):
            rows.setdefault(k, []).append(r)
        if sorted(rows) != list(range(len(rows))):
            continue
        if any(sum(lengths[r] for r in rs) > L for rs in rows.values()):
            continue
        for perm in itertools.product(*[list(itertools.permutations(rows[k]))
                                        for k in sorted(rows)]):
            req_row = np.zeros(n, np.int32)
            req_col = np.zeros(n, np.int32)
            for k, order in enumerate(perm):
                c = 0
                for r in order:
                    req_row[r], req_col[r] = k, c
                    c += lengths[r]
            lay = oracle.layout(lengths, req_row, req_col, len(rows), L)
            x = oracle.encoder_rows(cfg, w, names, ids, lay, L)
            out = oracle.unpack(x, lay["tok_index"], int(lengths.sum()))
            assert np.array_equal(out, ref)
            cnt += 1
    assert cnt > 50


def test_without_mask_or_restart_results_change():
    """Sanity: the invariant is not vacuous -- a dense (unmasked) row changes outputs."""
    cfg, w, names = _toy(seed=4)
    lengths = np.array([6, 9], np.int32)
    ids = wl.draw_token_ids(15, cfg.vocab, 2)
    res = oracle.run(cfg, w, names, lengths, ids, 16)
    lay = dict(res["layout"])
    seg = lay["segment_ids"].copy()
    seg[seg >= 0] = 0                      # one big segment = no mask (default inference)
    lay["segment_ids"] = seg
    x = oracle.encoder_rows(cfg, w, names, ids, lay, 16)
    out = oracle.unpack(x, lay["tok_index"], 15)
    assert not np.allclose(out, res["out"], atol=1e-3)


def test_qtile_intervals_match_brute_force_tile_enumeration():
    """P9: for L % 128 == 0, key tiles intersecting a q-tile's [lo, hi) are exactly the
    tiles holding some (query, key) pair of the same segment."""
    rng = np.random.default_rng(21)
    for L in (128, 256):
        lengths = wl.draw_lengths("paracrawl", 60, 3)
        lengths = np.minimum(lengths, L).astype(np.int32)
        pk = oracle.pack(lengths, L, 0)
        lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, 128)
        seg = lay["segment_ids"]
        M = len(seg)
        T = 128
        for t, (lo, hi) in enumerate(lay["qtile_kv"]):
            q = seg[t * T:(t + 1) * T]
            need = set()
            for kt in range(M // T):
                k = seg[kt * T:(kt + 1) * T]
                qs = set(q[q >= 0].tolist())
                if qs & set(k[k >= 0].tolist()):
                    need.add(kt)
            got = set() if lo < 0 else set(range(lo // T, (hi - 1) // T + 1))
            assert got == need, (L, t)
