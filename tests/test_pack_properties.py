"""Property-based tests (hypothesis) of the host packers: tcb_pack / tcb_pack_slotted (C++)
are bit-exact against the oracle packers + layout on generated inputs (packer
tests), and every packing satisfies the paper's constraints (10)-(11): each
request at most once, each row's words <= L, requests contiguous and non-overlapping."""
import numpy as np
import pytest

hyp = pytest.importorskip("hypothesis")
from hypothesis import given, settings, strategies as st  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icpp_fuc0z22_b200 as tcb  # noqa: E402


@st.composite
def pack_inputs(draw):
    L = draw(st.sampled_from([8, 16, 24, 32, 64, 128, 256, 512]))
    lengths = draw(st.lists(st.integers(1, L), min_size=0, max_size=120))
    max_rows = draw(st.sampled_from([0, 0, 1, 2, 5, 17]))
    policy = draw(st.sampled_from(list(oracle.POLICIES)))
    return np.asarray(lengths, np.int32), L, max_rows, policy


def _check_constraints(lengths, L, a, num_rows):
    placed = a["req_row"] >= 0
    used = np.zeros((num_rows, L), np.int32)
    for r in np.nonzero(placed)[0]:
        row, col, l = a["req_row"][r], a["req_col"][r], lengths[r]
        assert 0 <= col and col + l <= L                           # (11): fits in the row
        assert not used[row, col:col + l].any()                    # (10): no overlap / reuse
        used[row, col:col + l] = 1
    assert int(used.sum()) == int(lengths[placed].sum())


@settings(max_examples=300, deadline=None)
@given(pack_inputs())
def test_pack_bit_exact_and_feasible(inp):
    lengths, L, max_rows, policy = inp
    plan = tcb.tcb_pack(lengths, L, max_rows, policy)
    pk = oracle.pack(lengths, L, max_rows, policy)
    a = plan.arrays()
    assert plan.info["num_rows"] == pk["num_rows"]
    assert a["req_row"].tolist() == pk["req_row"].tolist()
    assert a["req_col"].tolist() == pk["req_col"].tolist()
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, 128)
    for k in ("seg_req", "seg_start", "cu_seqlens", "segment_ids", "positions", "qtile_kv"):
        assert a[k].tolist() == lay[k].tolist(), k
    if max_rows:
        assert plan.info["num_rows"] <= max_rows
    _check_constraints(lengths, L, a, plan.info["num_rows"])


@settings(max_examples=200, deadline=None)
@given(pack_inputs(), st.integers(0, 64))
def test_pack_slotted_bit_exact_and_within_slots(inp, z):
    lengths, L, max_rows, _ = inp
    z = min(z, L)
    plan = tcb.tcb_pack_slotted(lengths, L, z, max_rows)
    pk = oracle.pack_slotted(lengths, L, z, max_rows)
    a = plan.arrays()
    assert plan.info["slot_len"] == pk["slot_len"]
    assert a["req_row"].tolist() == pk["req_row"].tolist()
    assert a["req_col"].tolist() == pk["req_col"].tolist()
    _check_constraints(lengths, L, a, plan.info["num_rows"])
    zz = pk["slot_len"]
    for r in np.nonzero(a["req_row"] >= 0)[0]:                  # R26: never straddles a slot
        c, l = a["req_col"][r], lengths[r]
        assert c // zz == (c + l - 1) // zz and (c + l) <= (L // zz) * zz
