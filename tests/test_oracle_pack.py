"""Pins P1 / P2 of the oracle's packing and layout (o1) -- DESIGN.md §4.

The paper fixes: each request goes to at most one row (constraint (10)),
each row holds at most L words (constraint (11)), requests are put into
rows greedily (Alg. 1; reading R14 = First-Fit in input order), and
positions restart per request (separate PE).  These tests check the
oracle against properties that characterise those rules (not against a re-typed copy of
the oracle's loop), against exhaustive enumeration, and against the hand-derived
fixture tests/golden/f1_layout.json.
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle


def _expand(spec):
    out = []
    for tok in spec.split():
        if "x" in tok:
            v, c = tok.split("x")
            out += [int(v)] * int(c)
        else:
            a, b = tok.split("..")
            out += list(range(int(a), int(b) + 1))
    return out


def test_f1_golden_fixture(golden_dir):
    f1 = json.load(open(os.path.join(golden_dir, "f1_layout.json")))
    pk = oracle.pack(f1["lengths"], f1["row_len"], 0, f1["policy"])
    assert pk["num_rows"] == f1["num_rows"]
    assert pk["req_row"].tolist() == f1["req_row"]
    assert pk["req_col"].tolist() == f1["req_col"]
    lay = oracle.layout(f1["lengths"], pk["req_row"], pk["req_col"], pk["num_rows"],
                        f1["row_len"])
    assert lay["seg_req"].tolist() == f1["seg_req"]
    assert lay["seg_start"].tolist() == f1["seg_start"]
    assert lay["cu_seqlens"].tolist() == f1["cu_seqlens"]
    L = f1["row_len"]
    assert lay["segment_ids"][:L].tolist() == _expand(f1["segment_ids_row0"])
    assert lay["segment_ids"][L:].tolist() == _expand(f1["segment_ids_row1"])
    assert lay["positions"][:L].tolist() == _expand(f1["positions_row0"])
    assert lay["positions"][L:].tolist() == _expand(f1["positions_row1"])
    assert lay["qtile_kv"].tolist() == f1["qtile_kv_128"]
    pad = 1 - sum(f1["lengths"]) / (pk["num_rows"] * L)
    assert pad == f1["pad_fraction"]


def _check_feasible(lengths, pk, row_len, max_rows):
    """Constraints (10)-(11) + contiguity + conservation."""
    n = len(lengths)
    rows = pk["num_rows"]
    if max_rows:
        assert rows <= max_rows
    fill = np.zeros(rows, np.int64)
    cover = np.zeros((rows, row_len), np.int32)
    for r in range(n):
        if pk["req_row"][r] < 0:
            assert pk["req_col"][r] == -1
            continue
        k, c = pk["req_row"][r], pk["req_col"][r]
        assert 0 <= k < rows and 0 <= c and c + lengths[r] <= row_len     # (11)
        cover[k, c:c + lengths[r]] += 1
        fill[k] += lengths[r]
    assert cover.max(initial=0) <= 1                                        # no overlap
    # every row starts at column 0 and is contiguous (padding only at the tail, Fig. 1(c))
    for k in range(rows):
        assert cover[k, :fill[k]].all() and not cover[k, fill[k]:].any()
    placed = pk["req_row"] >= 0
    assert int(np.sum(lengths[placed])) == int(fill.sum())                 # conservation


def _check_first_fit(lengths, order, pk, row_len):
    """First-Fit characterisation: request r sits in row k only if, when r was placed,
    no lower row had room; and within a row, requests appear in placement order."""
    pos_in_order = {r: t for t, r in enumerate(order)}
    for r in order:
        k = pk["req_row"][r]
        if k < 0:
            continue
        earlier = [q for q in order[:pos_in_order[r]] if pk["req_row"][q] >= 0]
        for kk in range(k):
            used = sum(lengths[q] for q in earlier if pk["req_row"][q] == kk)
            assert row_len - used < lengths[r], (r, k, kk)
        same_row_before = sum(lengths[q] for q in earlier if pk["req_row"][q] == k)
        assert pk["req_col"][r] == same_row_before


@pytest.mark.parametrize("seed", range(40))
def test_first_fit_characterisation(seed):
    rng = np.random.default_rng(1000 + seed)
    L = int(rng.choice([8, 16, 32, 64]))
    n = int(rng.integers(1, 30))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    for max_rows in (0, 3):
        pk = oracle.pack(lengths, L, max_rows, "first_fit")
        _check_feasible(lengths, pk, L, max_rows)
        _check_first_fit(lengths, list(range(n)), pk, L)
        if max_rows == 0:
            assert (pk["req_row"] >= 0).all()
        else:  # an unplaced request fits in no row at the time it was considered
            for r in np.nonzero(pk["req_row"] < 0)[0]:
                used = [sum(lengths[q] for q in range(r) if pk["req_row"][q] == k)
                        for k in range(pk["num_rows"])]
                assert pk["num_rows"] == max_rows and all(L - u < lengths[r] for u in used)


@pytest.mark.parametrize("seed", range(20))
def test_ffd_next_fit_naive_sorted(seed):
    rng = np.random.default_rng(2000 + seed)
    L = 32
    n = int(rng.integers(1, 25))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    # FFD = First-Fit over the stable descending-length order
    pk = oracle.pack(lengths, L, 0, "first_fit_decreasing")
    order = sorted(range(n), key=lambda r: (-lengths[r], r))
    _check_feasible(lengths, pk, L, 0)
    _check_first_fit(lengths, order, pk, L)
    # Next-Fit: rows are opened in order; a new row only when the request did not fit the
    # open one
    pk = oracle.pack(lengths, L, 0, "next_fit")
    _check_feasible(lengths, pk, L, 0)
    rows = pk["req_row"]
    assert rows[0] == 0 and all(rows[i] - rows[i - 1] in (0, 1) for i in range(1, n))
    for i in range(1, n):
        if rows[i] == rows[i - 1] + 1:
            used = sum(lengths[q] for q in range(i) if rows[q] == rows[i - 1])
            assert L - used < lengths[i]
    # Naive: one request per row, in input order (R17); length-sorted: ascending, stable (R18)
    pk = oracle.pack(lengths, L, 0, "naive")
    assert pk["req_row"].tolist() == list(range(n)) and (pk["req_col"] == 0).all()
    pk = oracle.pack(lengths, L, 0, "length_sorted")
    order = sorted(range(n), key=lambda r: (lengths[r], r))
    assert [pk["req_row"][r] for r in order] == list(range(n))


def _bin_packing_opt(lengths, L):
    """Exhaustive optimum number of rows (set partitions), n <= 10."""
    n = len(lengths)
    best = n

    def rec(i, bins):
        nonlocal best
        if len(bins) >= best:
            return
        if i == n:
            best = len(bins)
            return
        for b in range(len(bins)):
            if bins[b] + lengths[i] <= L:
                bins[b] += lengths[i]
                rec(i + 1, bins)
                bins[b] -= lengths[i]
        bins.append(lengths[i])
        rec(i + 1, bins)
        bins.pop()

    rec(0, [])
    return best


@pytest.mark.parametrize("seed", range(25))
def test_first_fit_within_textbook_bound(seed):
    """FF <= floor(1.7 OPT) (Dosa & Sgall 2013; a textbook bound, not from the paper)."""
    rng = np.random.default_rng(3000 + seed)
    L = 16
    n = int(rng.integers(2, 11))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    opt = _bin_packing_opt(list(lengths), L)
    ff = oracle.pack(lengths, L, 0, "first_fit")["num_rows"]
    assert opt <= ff <= int(np.floor(1.7 * opt))


def _brute_layout(lengths, req_row, req_col, rows, L, qtile):
    """P1: for each slot scan every request to find the one covering it."""
    M = rows * L
    n = len(lengths)
    cu_req = np.concatenate([[0], np.cumsum(lengths)])
    seg_ids, pos, tok = [-1] * M, [-1] * M, [-1] * M
    owners = []
    for s in range(M):
        k, c = divmod(s, L)
        owner = [r for r in range(n) if req_row[r] == k and req_col[r] <= c < req_col[r] + lengths[r]]
        assert len(owner) <= 1
        owners.append(owner[0] if owner else -1)
    # segments: maximal runs of equal owner, numbered in slot order
    seg_req, seg_start = [], []
    for s in range(M):
        r = owners[s]
        if r < 0:
            continue
        if s == 0 or owners[s - 1] != r or s % L == 0:
            seg_req.append(r)
            seg_start.append(s)
        seg_ids[s] = len(seg_req) - 1
        pos[s] = s - seg_start[-1]
        tok[s] = int(cu_req[r]) + pos[s]
    cu = [0]
    for r in seg_req:
        cu.append(cu[-1] + int(lengths[r]))
    nt = (M + qtile - 1) // qtile
    qkv = []
    for t in range(nt):
        real = [s for s in range(t * qtile, min(M, (t + 1) * qtile)) if seg_ids[s] >= 0]
        if not real:
            qkv.append([-1, -1])
        else:
            a, b = seg_ids[real[0]], seg_ids[real[-1]]
            qkv.append([seg_start[a], seg_start[b] + int(lengths[seg_req[b]])])
    return dict(segment_ids=seg_ids, positions=pos, tok_index=tok, seg_req=seg_req,
                seg_start=seg_start, cu_seqlens=cu, qtile_kv=qkv)


@pytest.mark.parametrize("policy", list(oracle.POLICIES))
@pytest.mark.parametrize("seed", range(6))
def test_layout_matches_brute_force_scan(policy, seed):
    rng = np.random.default_rng(4000 + seed)
    L = int(rng.choice([16, 32, 48]))
    n = int(rng.integers(1, 20))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    max_rows = int(rng.choice([0, 4]))
    pk = oracle.pack(lengths, L, max_rows, policy)
    for qtile in (16, 128):
        lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, qtile)
        ref = _brute_layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, qtile)
        for key in ("segment_ids", "positions", "tok_index", "seg_req", "seg_start",
                    "cu_seqlens"):
            assert lay[key].tolist() == ref[key], key
        assert lay["qtile_kv"].tolist() == ref["qtile_kv"]


def test_pack_errors_and_empty():
    with pytest.raises(oracle.OracleError) as e:
        oracle.pack([5, 40], 32)
    assert e.value.code == -2                       # R15: longer than a row
    with pytest.raises(oracle.OracleError) as e:
        oracle.pack([5, 0], 32)
    assert e.value.code == -1
    pk = oracle.pack([], 32)
    assert pk["num_rows"] == 0
    lay = oracle.layout([], pk["req_row"], pk["req_col"], 0, 32)
    assert lay["num_segments"] == 0 and len(lay["segment_ids"]) == 0
    # exactly full rows: no padding
    pk = oracle.pack([32, 16, 16], 32)
    assert pk["num_rows"] == 2 and pk["req_row"].tolist() == [0, 1, 1]
