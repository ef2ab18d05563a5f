"""CPU tests of the C ABI (no GPU needed): libtcb.so loads and exports every declared
symbol; the C++ packer (tcb_pack) is bit-exact against the oracle's packer and layout on
random and golden inputs, for every policy; error conventions; plan counters against a
brute-force tile enumeration (P9); device calls without a GPU fail loudly (no fallback).
"""
import json
import os
import re

import numpy as np
import pytest

import oracle
import tcb_workload as wl
import paper_conf_icpp_fuc0z22_b200 as tcb
from paper_conf_icpp_fuc0z22_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    names = set()
    for h in ("tcb.h", "tcb_ops.h", "tcb_decoder.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names |= set(re.findall(r"\b(tcb_[a-z_0-9]+)\s*\(", src))
    return names


def test_library_exports_every_declared_symbol():
    L = _lib.lib()
    declared = _declared_symbols()
    assert declared == set(_lib.EXPORTS), declared ^ set(_lib.EXPORTS)
    for name in declared:
        assert hasattr(L, name), name
    assert b"sm_100a" in L.tcb_version()


def _plan_vs_oracle(lengths, L, max_rows, policy):
    plan = tcb.tcb_pack(lengths, L, max_rows, policy)
    pk = oracle.pack(lengths, L, max_rows, policy)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, 128)
    a = plan.arrays()
    assert plan.info["num_rows"] == pk["num_rows"]
    assert a["req_row"].tolist() == pk["req_row"].tolist()
    assert a["req_col"].tolist() == pk["req_col"].tolist()
    for k in ("seg_req", "seg_start", "cu_seqlens", "segment_ids", "positions"):
        assert a[k].tolist() == lay[k].tolist(), k
    assert a["qtile_kv"].tolist() == lay["qtile_kv"].tolist()
    return plan, lay


@pytest.mark.parametrize("policy", list(oracle.POLICIES))
@pytest.mark.parametrize("seed", range(12))
def test_pack_bit_exact_vs_oracle_random(policy, seed):
    rng = np.random.default_rng(500 + seed)
    L = int(rng.choice([8, 32, 64, 128, 256]))
    n = int(rng.integers(0, 200))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    max_rows = int(rng.choice([0, 0, 3, 20]))
    _plan_vs_oracle(lengths, L, max_rows, policy)


@pytest.mark.parametrize("dist,L", [("paracrawl", 128), ("dia", 512), ("mixed_8_512", 512),
                                    ("wmt", 256), ("paper_normal_20", 128)])
def test_pack_bit_exact_vs_oracle_workloads(dist, L):
    lengths = np.minimum(wl.draw_lengths(dist, 800, 77), L).astype(np.int32)
    _plan_vs_oracle(lengths, L, 64, "first_fit")


def test_pack_golden_f1(golden_dir):
    f1 = json.load(open(os.path.join(golden_dir, "f1_layout.json")))
    plan = tcb.tcb_pack(f1["lengths"], f1["row_len"])
    a = plan.arrays()
    assert a["req_row"].tolist() == f1["req_row"]
    assert a["req_col"].tolist() == f1["req_col"]
    assert a["seg_start"].tolist() == f1["seg_start"]
    assert a["cu_seqlens"].tolist() == f1["cu_seqlens"]
    assert a["qtile_kv"].tolist() == f1["qtile_kv_128"]
    st = plan.segtab()
    assert st[:4].tolist() == [8, 64, 32, 58]
    assert len(st) == 4 * 9 + 4 + 4
    assert st[36:39].tolist() == [0, 3, 8]          # row_first: row 0 -> seg 0, row 1 -> 3, end
    assert st[40] == 0                              # query-block order: the single q-block
    recs = st[4:36].reshape(-1, 4)
    assert recs[:, 0].tolist() == f1["seg_start"]
    assert recs[:, 1].tolist() == [f1["lengths"][r] for r in f1["seg_req"]]
    cu_req = np.concatenate([[0], np.cumsum(f1["lengths"])])
    assert recs[:, 2].tolist() == [int(cu_req[r]) for r in f1["seg_req"]]
    assert recs[:, 3].tolist() == f1["seg_req"]
    assert plan.info["placed_tokens"] == 58 and plan.info["num_slots"] == 64


def _slotted_vs_oracle(lengths, L, z, max_rows):
    plan = tcb.tcb_pack_slotted(lengths, L, z, max_rows)
    pk = oracle.pack_slotted(lengths, L, z, max_rows)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L, 128)
    a = plan.arrays()
    assert plan.info["slot_len"] == pk["slot_len"]
    assert plan.info["num_rows"] == pk["num_rows"]
    assert a["req_row"].tolist() == pk["req_row"].tolist()
    assert a["req_col"].tolist() == pk["req_col"].tolist()
    for k in ("seg_req", "seg_start", "cu_seqlens", "segment_ids", "positions"):
        assert a[k].tolist() == lay[k].tolist(), k
    assert a["qtile_kv"].tolist() == lay["qtile_kv"].tolist()
    return plan


@pytest.mark.parametrize("seed", range(16))
def test_pack_slotted_bit_exact_vs_oracle_random(seed):
    rng = np.random.default_rng(900 + seed)
    L = int(rng.choice([8, 32, 64, 128, 256]))
    n = int(rng.integers(0, 200))
    lengths = rng.integers(1, L + 1, size=n).astype(np.int32)
    max_rows = int(rng.choice([0, 0, 3, 20]))
    for z in (0, int(rng.integers(1, L + 1)), L):
        _slotted_vs_oracle(lengths, L, z, max_rows)


@pytest.mark.parametrize("dist,L,slots", [("paracrawl", 128, (2, 4)), ("dia", 512, (2, 4, 7)),
                                          ("paper_normal_20", 128, (2, 3, 6))])
def test_pack_slotted_bit_exact_vs_oracle_workloads(dist, L, slots):
    lengths = np.minimum(wl.draw_lengths(dist, 800, 78), L).astype(np.int32)
    for s in slots:
        _slotted_vs_oracle(lengths, L, L // s, 64)


def test_pack_slotted_golden_f1s(golden_dir):
    f = json.load(open(os.path.join(golden_dir, "f1s_slotted.json")))
    for c in f["cases"]:
        plan = tcb.tcb_pack_slotted(f["lengths"], f["row_len"], c["slot_len_arg"])
        a = plan.arrays()
        assert plan.info["slot_len"] == c["slot_len"]
        assert a["req_row"].tolist() == c["req_row"]
        assert a["req_col"].tolist() == c["req_col"]
        assert a["seg_req"].tolist() == c["seg_req"]
        assert a["seg_start"].tolist() == c["seg_start"]
        assert a["cu_seqlens"].tolist() == c["cu_seqlens"]
        assert a["qtile_kv"].tolist() == c["qtile_kv_128"]
        st = plan.segtab()
        S = len(c["seg_req"])
        recs = st[4:4 + 4 * S].reshape(-1, 4)
        assert recs[:, 0].tolist() == c["seg_start"]
        assert recs[:, 3].tolist() == c["seg_req"]


def test_pack_slotted_errors():
    with pytest.raises(tcb.TcbError) as e:
        tcb.tcb_pack_slotted([3, 40], 32, 8)
    assert e.value.status == -2
    with pytest.raises(tcb.TcbError) as e:
        tcb.tcb_pack_slotted([3], 32, 33)
    assert e.value.status == -1
    with pytest.raises(tcb.TcbError) as e:
        tcb.tcb_pack_slotted([3], 32, -1)
    assert e.value.status == -1
    p = tcb.tcb_pack_slotted([9, 4], 32, 8)          # 9 > z: deferred, not an error
    assert p.arrays()["req_row"].tolist() == [-1, 0]
    assert tcb.tcb_pack([3], 32).info["slot_len"] == 0


def test_pack_errors():
    with pytest.raises(tcb.TcbError) as e:
        tcb.tcb_pack([3, 40], 32)
    assert e.value.status == -2 and "request 1" in str(e.value)
    with pytest.raises(tcb.TcbError) as e:
        tcb.tcb_pack([3, 0], 32)
    assert e.value.status == -1
    with pytest.raises(tcb.TcbError) as e:
        tcb.tcb_pack([3], 30)          # row_len % 8 != 0
    assert e.value.status == -1
    with pytest.raises(tcb.TcbError):
        tcb.tcb_pack([3], 32, -1)
    p = tcb.tcb_pack([], 32)
    assert p.info["num_rows"] == 0 and p.info["num_slots"] == 0
    assert p.segtab().tolist() == [0, 0, 32, 0, 0, 0, 0, 0]


def test_plan_counters_vs_brute_force():
    """P9 on the product's plan counters: 128x128 tiles touching a diagonal block, the
    dense count, sum l^2, and the tcgen05 attention kernel's executed S elements and softmax
    elements (re-derived here from its stated geometry: 128-query items, 128-key chunks from
    the item's interval start rounded down to 8, 32-row x 32-key softmax liveness groups)."""
    lengths = np.minimum(wl.draw_lengths("dia", 300, 5), 512).astype(np.int32)
    plan = tcb.tcb_pack(lengths, 512, 16)
    a = plan.arrays()
    seg = a["segment_ids"]
    M = len(seg)
    T = 128
    visited = 0
    for qt in range(M // T):
        q = set(seg[qt * T:(qt + 1) * T].tolist()) - {-1}
        for kt in range(M // T):
            k = set(seg[kt * T:(kt + 1) * T].tolist()) - {-1}
            if (qt * T) // 512 == (kt * T) // 512 and q & k:
                visited += 1
    info = plan.info
    assert info["kv_tiles_visited"] == visited
    assert info["kv_tiles_dense"] == info["num_rows"] * 16
    placed = a["req_row"] >= 0
    assert info["useful_score_elems"] == int(np.sum(lengths[placed].astype(np.int64) ** 2))
    starts, lens = a["seg_start"], lengths[a["seg_req"]]
    ex = sm = 0
    for q0 in range(0, M, 128):
        iv = []
        for g in range(4):
            ss = [s for s in seg[q0 + 32 * g:q0 + 32 * g + 32] if s >= 0]
            iv.append((min(starts[s] for s in ss), max(starts[s] + lens[s] for s in ss))
                      if ss else None)
        real = [x for x in iv if x]
        if not real:
            continue
        lo, hi = min(x[0] for x in real), max(x[1] for x in real)
        kb = lo - lo % 8
        nch = -(-(hi - kb) // 128)
        ex += nch * 128 * 128
        for x in real:
            sm += 32 * 32 * sum(1 for gk in range(kb, kb + 128 * nch, 32)
                                if gk < x[1] and gk + 32 > x[0])
    assert info["executed_score_elems"] == ex
    assert info["softmax_score_elems"] == sm
    assert info["useful_score_elems"] <= sm <= ex


def test_device_calls_fail_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is visible")
    m = wl.MODELS["toy"]
    cfg = _lib.ModelConfig(m.num_layers, m.d_model, m.num_heads, m.d_ff, m.vocab, m.max_pos,
                           0, 0, 0, 0, 0, 1e-5, 1e-5, 1.0)
    import ctypes
    n = _lib.lib().tcb_weights_count(ctypes.byref(cfg))
    assert n == 5 + 12 * m.num_layers
    fake = (ctypes.c_void_p * n)(*([4096] * n))
    h = ctypes.c_void_p()
    st = _lib.lib().tcb_weights_create(ctypes.byref(cfg), fake, n, ctypes.byref(h))
    assert st == -7   # TCB_ERR_NO_DEVICE: there is no CPU fallback
    assert b"no CPU fallback" in _lib.lib().tcb_last_error()
    st = _lib.lib().tcb_op_linear(1, 128, 64, 64, 4096, 4096, 4096, None, 0, 4096, None)
    assert st == -7


def test_decoder_abi_validates_without_a_gpu():
    """f4 ABI (include/tcb_decoder.h): weight count, NULL checks, no CPU fallback."""
    import ctypes
    import tcb_workload as wl
    m = wl.MODELS["transformer-base"]
    cfg = _lib.ModelConfig(m.num_layers, m.d_model, m.num_heads, m.d_ff, m.vocab, m.max_pos, 1,
                           1, 0, 0, 0, m.ln_eps, m.emb_ln_eps, m.emb_scale)
    L = _lib.lib()
    assert L.tcb_decoder_weights_count(ctypes.byref(cfg)) == 20 * m.num_layers
    h = ctypes.c_void_p()
    assert L.tcb_decoder_create(None, None, 0, 1, 1, 1, ctypes.byref(h)) == -1
    assert L.tcb_decode_greedy(None, None, None, 1, None, None, None) == -1
    st = _lib.DecodeStats()
    assert L.tcb_decoder_stats(None, ctypes.byref(st)) == -1
    assert len(wl.dec_weight_names(m)) == 20 * m.num_layers


@pytest.mark.parametrize("dist,L,B,seed", [("dia", 512, 16, 3), ("paracrawl", 128, 64, 4),
                                           ("mixed_8_512", 512, 16, 5), ("wmt", 256, 32, 6)])
def test_segtab_query_block_order(dist, L, B, seed):
    """The segment table's query-block order (attention work order): a permutation of the
    q-blocks, chunk counts non-increasing, ties by index -- chunk counts re-derived here from
    the layout (128-key chunks from the block's interval start rounded down to 8)."""
    lengths = np.minimum(wl.draw_lengths(dist, 4 * B, seed), L).astype(np.int32)
    plan = tcb.tcb_pack(lengths, L, B)
    a = plan.arrays()
    seg, starts, lens = a["segment_ids"], a["seg_start"], lengths[a["seg_req"]]
    M = len(seg)
    QT = -(-M // 128)
    S = len(a["seg_req"])
    st = plan.segtab()
    off = 4 * (1 + S) + (plan.info["num_rows"] + 1 + 3) // 4 * 4
    order = st[off:off + QT].tolist()
    assert len(st) == off + (QT + 3) // 4 * 4
    nch = []
    for t in range(QT):
        ss = [s for s in seg[t * 128:(t + 1) * 128] if s >= 0]
        if not ss:
            nch.append(0)
            continue
        lo, hi = min(starts[s] for s in ss), max(starts[s] + lens[s] for s in ss)
        kb = lo - lo % 8
        nch.append(-(-(hi - kb) // 128))
    assert sorted(order) == list(range(QT))
    keys = [(-nch[q], q) for q in order]
    assert keys == sorted(keys)
