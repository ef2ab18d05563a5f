"""Pins of the oracle's slotted ConcatBatching packer (§8(f) row f1) -- DESIGN.md §4.

§4.2 divides each row into slots, Eq. (8) computes attention per slot,
and Alg. 2 sets the slot size z to the largest length (l.4), divides
each row into slots of z (l.5) and puts requests into slots greedily (l.7); pure
ConcatBatching is "a special case whose slot size is equal to the batch length L"
(PAPER.md:1426-1428).  Reading R26: First-Fit over slots in row-major order, floor(L/z)
slots per row, requests never straddle a slot, requests that fit nowhere are deferred.

Pins: the hand-derived fixture tests/golden/f1s_slotted.json; z = L reduces exactly to
the (separately pinned) First-Fit packer; all-equal lengths have a closed form; the
First-Fit-over-slots characterisation on random inputs; and the method's invariant that
every request's encoder output is bitwise the one it gets alone (P4) under slotted packing.
"""
import json
import os

import numpy as np
import pytest

import oracle
import tcb_workload as wl

from test_oracle_pack import _expand, _brute_layout


def _fixture(golden_dir):
    return json.load(open(os.path.join(golden_dir, "f1s_slotted.json")))


@pytest.mark.parametrize("case", [0, 1])
def test_f1s_golden_fixture(golden_dir, case):
    f = _fixture(golden_dir)
    c = f["cases"][case]
    L = f["row_len"]
    pk = oracle.pack_slotted(f["lengths"], L, c["slot_len_arg"])
    assert pk["slot_len"] == c["slot_len"]
    assert pk["num_rows"] == c["num_rows"]
    assert pk["req_row"].tolist() == c["req_row"]
    assert pk["req_col"].tolist() == c["req_col"]
    lay = oracle.layout(f["lengths"], pk["req_row"], pk["req_col"], pk["num_rows"], L)
    for key in ("seg_req", "seg_start", "cu_seqlens"):
        assert lay[key].tolist() == c[key], key
    for k in range(pk["num_rows"]):
        assert lay["segment_ids"][k * L:(k + 1) * L].tolist() == _expand(c["segment_ids_rows"][k])
        assert lay["positions"][k * L:(k + 1) * L].tolist() == _expand(c["positions_rows"][k])
    assert lay["qtile_kv"].tolist() == c["qtile_kv_128"]
    assert 1 - sum(f["lengths"]) / (pk["num_rows"] * L) == pytest.approx(c["pad_fraction"], rel=1e-15)


@pytest.mark.parametrize("seed", range(20))
def test_slot_len_equal_row_len_is_first_fit(seed):
    rng = np.random.default_rng(7000 + seed)
    L = int(rng.choice([8, 16, 32, 128]))
    n = int(rng.integers(1, 60))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    for max_rows in (0, 2, 5):
        ff = oracle.pack(lengths, L, max_rows, "first_fit")
        sl = oracle.pack_slotted(lengths, L, L, max_rows)
        assert sl["slot_len"] == L
        assert sl["num_rows"] == ff["num_rows"]
        assert sl["req_row"].tolist() == ff["req_row"].tolist()
        assert sl["req_col"].tolist() == ff["req_col"].tolist()


@pytest.mark.parametrize("L,z,n", [(32, 8, 9), (128, 32, 17), (128, 40, 7), (64, 64, 3)])
def test_equal_lengths_closed_form(L, z, n):
    """All lengths == z: request i occupies slot i, i.e. row i // floor(L/z) at column
    (i % floor(L/z)) * z."""
    per = L // z
    pk = oracle.pack_slotted([z] * n, L, 0)
    assert pk["slot_len"] == z
    assert pk["num_rows"] == -(-n // per)
    assert pk["req_row"].tolist() == [i // per for i in range(n)]
    assert pk["req_col"].tolist() == [(i % per) * z for i in range(n)]


def _check_slotted(lengths, pk, L, max_rows):
    """Feasibility + the First-Fit-over-slots characterisation, from the outputs only."""
    z = pk["slot_len"]
    per = L // z
    n = len(lengths)
    rows = pk["num_rows"]
    if max_rows:
        assert rows <= max_rows
    fill = {}
    cover = np.zeros((rows, L), np.int32)
    for r in range(n):
        k, c = int(pk["req_row"][r]), int(pk["req_col"][r])
        l = int(lengths[r])
        if k < 0:
            assert c == -1
            # deferred: longer than a slot, or no slot had room and no row could be opened
            if l <= z:
                assert max_rows and all(z - fill.get(s, 0) < l for s in range(max_rows * per))
            continue
        s = k * per + c // z
        assert c // z < per and (c + l - 1) // z == c // z          # never straddles a slot
        assert c % z == fill.get(s, 0)                                # contiguous in the slot
        # First-Fit: no earlier slot (already open or in an opened row) had room
        for s2 in range(s):
            assert z - fill.get(s2, 0) < l, (r, s, s2)
        fill[s] = fill.get(s, 0) + l
        cover[k, c:c + l] += 1
    assert cover.max(initial=0) <= 1
    placed = pk["req_row"] >= 0
    assert int(np.sum(lengths[placed])) == int(cover.sum())
    # no empty row was opened
    assert all(cover[k].any() for k in range(rows))


@pytest.mark.parametrize("seed", range(30))
def test_first_fit_over_slots_characterisation(seed):
    rng = np.random.default_rng(8000 + seed)
    L = int(rng.choice([16, 32, 64, 128]))
    n = int(rng.integers(1, 40))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    for z in (0, int(rng.integers(1, L + 1)), L // 2 or 1):
        for max_rows in (0, 3):
            pk = oracle.pack_slotted(lengths, L, z, max_rows)
            if z:
                assert pk["slot_len"] == z
            else:
                assert pk["slot_len"] == int(lengths.max())
            _check_slotted(lengths, pk, L, max_rows)
            lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, 16)
            ref = _brute_layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, 16)
            for key in ("segment_ids", "positions", "tok_index", "seg_req", "seg_start"):
                assert lay[key].tolist() == ref[key], key


def test_longer_than_slot_deferred_and_errors():
    pk = oracle.pack_slotted([5, 9, 4], 16, 8)
    assert pk["req_row"].tolist() == [0, -1, 0]
    assert pk["req_col"].tolist() == [0, -1, 8]
    with pytest.raises(oracle.OracleError) as e:
        oracle.pack_slotted([5, 40], 32, 8)
    assert e.value.code == -2
    with pytest.raises(oracle.OracleError):
        oracle.pack_slotted([5], 32, 33)
    pk = oracle.pack_slotted([], 32, 0)
    assert pk["num_rows"] == 0


def test_slotted_outputs_equal_alone_bitwise():
    """P4 under slotted packing: per-request outputs are bitwise those of pure Concat FF
    (which test_oracle_invariants pins to the request-alone result)."""
    cfg = wl.ModelConfig("t", 2, 64, 2, 256, 128, 64, "fp32", "gelu", "sin_paper", False,
                         False, 1e-5, 1e-5, 1.0)
    w, names = wl.draw_weights(cfg, 2), wl.weight_names(cfg)
    lengths = wl.draw_lengths("uniform_3_16", 8, 0)
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 1)
    ref = oracle.run(cfg, w, names, lengths, ids, 32)["out"]
    for z in (0, 16, 20):
        res = oracle.run(cfg, w, names, lengths, ids, 32, policy="slotted", slot_len=z)
        assert np.array_equal(res["out"], ref), z
