"""Per-kernel parity of the CUDA path against the float64 oracle (GPU, sm_100a).

Each kernel is called through the C ABI (include/tcb.h, include/tcb_ops.h) on seeded
inputs; the oracle computes the same step in f64 on the identical (bf16-representable)
values.  Integer metadata must be bit-exact.
"""
import numpy as np
import pytest

import oracle
import tcb_workload as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_icpp_fuc0z22_b200 as tcb  # noqa: E402
from _helpers import small_model  # noqa: E402


def _dev(x, dtype=None):
    t = torch.from_numpy(np.ascontiguousarray(x))
    return t.to("cuda", dtype=dtype) if dtype is not None else t.to("cuda")


def _bf16(x):
    return wl.round_to_bf16(np.asarray(x, np.float32))


# ------------------------------------------------------------------------------ linear --
LIN_SHAPES = [(1, 64, 64), (100, 128, 64), (128, 256, 512), (1000, 192, 128),
              (4133, 1536, 512), (777, 768, 768), (2048, 512, 2048), (300, 3072, 1024)]


@pytest.mark.parametrize("M,N,K", LIN_SHAPES)
@pytest.mark.parametrize("epi", ["bias", "bias_gelu", "bias_relu", "bias_residual"])
def test_linear_bf16_tcgen05_vs_oracle(M, N, K, epi):
    rng = np.random.default_rng(M * 7 + N * 3 + K)
    A = _bf16(rng.normal(size=(M, K)))
    W = _bf16(rng.uniform(-1, 1, size=(N, K)) * np.sqrt(3.0 / K))
    b = _bf16(rng.normal(0, 0.1, size=N))
    R = _bf16(rng.normal(size=(M, N))) if epi == "bias_residual" else None
    out = tcb.op_linear(_dev(A, torch.bfloat16), _dev(W, torch.bfloat16), _dev(b, torch.float32),
                        _dev(R, torch.bfloat16) if R is not None else None, epi)
    torch.cuda.synchronize()
    got = out.float().cpu().numpy()
    act = {"bias_gelu": "gelu", "bias_relu": "relu"}.get(epi, "none")
    ref = oracle.linear(A, W, b, R, act)
    # one bf16 rounding of the output (2^-8 relative) + fp32 accumulation-order noise
    err = np.abs(got - ref)
    bound = 2.0 ** -8 * np.abs(ref) + 1e-3 * np.max(np.abs(ref)) + 1e-6
    assert np.all(err <= bound), float(np.max(err / bound))


@pytest.mark.parametrize("M,K,N", [(1, 512, 512), (300, 512, 512), (4133, 512, 512),
                                   (1000, 1024, 512), (1000, 2048, 512), (513, 4096, 512),
                                   (32768, 512, 512), (1, 768, 768), (777, 768, 768),
                                   (3001, 3072, 768), (32768, 768, 768), (32768, 3072, 768),
                                   (300, 1024, 1024), (2049, 4096, 1024),
                                   (1, 4096, 1024), (300, 2048, 1024), (32768, 1024, 1024),
                                   (32768, 4096, 1024),
                                   # tail split of the L2-exchange kernel (half-width units for
                                   # the row tiles after the last complete round), ragged M
                                   (32668, 2048, 512), (26000, 3072, 768)])
def test_linear_ln_fused_vs_oracle(M, K, N):
    """W_O / FFN2 + bias + residual + LayerNorm in one tcgen05 kernel (N = 512, 768, 1024:
    clusters of N / 256 CTA pairs exchanging the row statistics over DSMEM; N = 1024 with
    K >= 2048: single pairs exchanging them through L2)."""
    rng = np.random.default_rng(M + K + N)
    A = _bf16(rng.normal(size=(M, K)))
    W = _bf16(rng.uniform(-1, 1, size=(N, K)) * np.sqrt(3.0 / K))
    b = _bf16(rng.normal(0, 0.1, size=N))
    R = _bf16(rng.normal(size=(M, N)))
    g = _bf16(1 + rng.normal(0, 0.1, size=N))
    be = _bf16(rng.normal(0, 0.1, size=N))
    seg = np.zeros(M, np.int32)
    seg[::7] = -1
    out = tcb.op_linear_ln(_dev(A, torch.bfloat16), _dev(W, torch.bfloat16), _dev(b, torch.float32),
                           _dev(R, torch.bfloat16), _dev(g, torch.float32), _dev(be, torch.float32),
                           1e-5, _dev(seg))
    torch.cuda.synchronize()
    got = out.float().cpu().numpy()
    z = oracle.linear(A, W, b, R)
    ref = oracle.layernorm(z, g, be, 1e-5)
    real = seg >= 0
    err = np.abs(got[real] - ref[real])
    # one bf16 rounding of the output (2^-8 relative) + fp32 statistics / accumulation noise
    bound = 2.0 ** -8 * np.abs(ref[real]) + 1e-3
    assert np.all(err <= bound), float(np.max(err / bound))
    assert np.all(got[~real] == 0)


def test_linear_ln_cluster_kernel_at_d512():
    """The cluster kernel also serves N = 512 (TCB_LN_KERNEL=cluster, read once per process):
    checked in a subprocess so the default (single-pair) choice of this process stays."""
    import subprocess, sys, os
    code = ("import sys; sys.path.insert(0, 'tests'); import test_gpu_kernels as t; "
            "t.test_linear_ln_fused_vs_oracle(4133, 1024, 512); t.test_linear_ln_fused_vs_oracle(1, 512, 512)")
    env = dict(os.environ, TCB_LN_KERNEL="cluster")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                       cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]


def test_linear_ln_l2_exchange_kernel_everywhere():
    """TCB_LN_KERNEL=global runs the L2-exchange kernel for every N = 768 / 1024 shape
    (the default keeps the cluster kernel there): subprocess, the choice is read once."""
    import subprocess, sys, os
    code = ("import sys; sys.path.insert(0, 'tests'); import test_gpu_kernels as t; "
            "t.test_linear_ln_fused_vs_oracle(777, 768, 768); t.test_linear_ln_fused_vs_oracle(1, 768, 768); "
            "t.test_linear_ln_fused_vs_oracle(3001, 3072, 768); t.test_linear_ln_fused_vs_oracle(300, 1024, 1024)")
    env = dict(os.environ, TCB_LN_KERNEL="global")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                       cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]


def test_linear_ln_l2_exchange_without_tail_split():
    """TCB_LNG_TAIL=0: the L2-exchange kernel with full-width units only (the default splits
    the row tiles after the last complete round of the grid into half-width units)."""
    import subprocess, sys, os
    code = ("import sys; sys.path.insert(0, 'tests'); import test_gpu_kernels as t; "
            "t.test_linear_ln_fused_vs_oracle(32668, 2048, 512); t.test_linear_ln_fused_vs_oracle(26000, 3072, 768)")
    env = dict(os.environ, TCB_LNG_TAIL="0")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                       cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))), timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]


@pytest.mark.parametrize("M,N,K", [(64, 192, 64), (130, 256, 64), (37, 64, 256)])
@pytest.mark.parametrize("epi", ["bias", "bias_gelu", "bias_residual"])
def test_linear_f32_simt_vs_oracle(M, N, K, epi):
    rng = np.random.default_rng(11 + M + N + K)
    A = rng.normal(size=(M, K)).astype(np.float32)
    W = (rng.uniform(-1, 1, size=(N, K)) * np.sqrt(3.0 / K)).astype(np.float32)
    b = rng.normal(0, 0.1, size=N).astype(np.float32)
    R = rng.normal(size=(M, N)).astype(np.float32) if epi == "bias_residual" else None
    out = tcb.op_linear(_dev(A), _dev(W), _dev(b), _dev(R) if R is not None else None, epi)
    torch.cuda.synchronize()
    ref = oracle.linear(A, W, b, R, {"bias_gelu": "gelu"}.get(epi, "none"))
    assert np.max(np.abs(out.cpu().numpy() - ref)) <= 2e-5 * max(1.0, np.max(np.abs(ref)))


def test_linear_deterministic_and_m_zero():
    rng = np.random.default_rng(3)
    A = _dev(_bf16(rng.normal(size=(999, 512))), torch.bfloat16)
    W = _dev(_bf16(rng.normal(size=(1536, 512)) * 0.05), torch.bfloat16)
    b = _dev(np.zeros(1536, np.float32))
    o1 = tcb.op_linear(A, W, b)
    o2 = tcb.op_linear(A, W, b)
    torch.cuda.synchronize()
    assert torch.equal(o1, o2)
    e = tcb.op_linear(A[:0], W, b)
    assert e.shape == (0, 1536)


# --------------------------------------------------------------------------- attention --
def _attn_case(lengths, L, d, h, dtype, seed, max_rows=0):
    rng = np.random.default_rng(seed)
    plan = tcb.tcb_pack(lengths, L, max_rows)
    arr = plan.arrays()
    M = plan.num_slots
    qkv = rng.normal(size=(M, 3 * d)).astype(np.float32)
    if dtype == "bf16":
        qkv = _bf16(qkv)
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    seg = _dev(arr["segment_ids"])
    segtab = _dev(plan.segtab())
    out = tcb.op_attention(_dev(qkv, tdt), seg, segtab, h)
    torch.cuda.synchronize()
    ref = oracle.attention(qkv, arr["segment_ids"], plan.info["num_rows"], L, d, h)
    return out.float().cpu().numpy(), ref, arr["segment_ids"]


@pytest.mark.parametrize("case", [
    ("uniform_3_16", 40, 32), ("paracrawl", 300, 128), ("dia", 60, 512), ("wmt", 200, 256),
    ("mixed_8_512", 80, 512)])
def test_attention_bf16_vs_oracle(case):
    dist, n, L = case
    lengths = np.minimum(wl.draw_lengths(dist, n, 9), L).astype(np.int32)
    got, ref, seg = _attn_case(lengths, L, 256, 4, "bf16", 1)
    real = seg >= 0
    # P is rounded to bf16 before P.V and O to bf16 on store: ~2^-8 relative
    for s in np.unique(seg[real]):
        rows = seg == s
        e = np.max(np.abs(got[rows] - ref[rows])) / np.max(np.abs(ref[rows]))
        assert e <= 1.5e-2, (s, e)
    assert np.all(got[~real] == 0)


def test_attention_bf16_single_long_request_and_tail():
    """One request filling a 512 row (textbook SDPA) + a ragged last row + pad tail."""
    got, ref, seg = _attn_case(np.array([512, 77, 3], np.int32), 512, 128, 2, "bf16", 4)
    real = seg >= 0
    assert np.max(np.abs(got[real] - ref[real])) / np.max(np.abs(ref[real])) <= 1.5e-2
    assert np.all(got[~real] == 0)


def test_attention_bf16_running_max_rescale():
    """Scores that grow along the key axis force the online softmax to move its running
    maximum across 128-key chunks (the lazy O-rescale path) -- with a mix of rows that do
    and do not rescale inside the same warp."""
    rng = np.random.default_rng(17)
    lengths = np.array([500, 300, 200, 12], np.int32)
    L, d, h = 512, 128, 2
    plan = tcb.tcb_pack(lengths, L, 0)
    arr = plan.arrays()
    M = plan.num_slots
    qkv = rng.normal(size=(M, 3 * d)).astype(np.float32)
    pos = np.maximum(arr["positions"], 0).astype(np.float32)
    qkv[:, :d] *= 2.0
    qkv[:, d:2 * d] *= (1.0 + pos / 40.0)[:, None]      # key norms grow with position
    qkv[::3, :d] *= 0.05                                 # some rows never rescale
    qkv = _bf16(qkv)
    out = tcb.op_attention(_dev(qkv, torch.bfloat16), _dev(arr["segment_ids"]),
                           _dev(plan.segtab()), h)
    torch.cuda.synchronize()
    got = out.float().cpu().numpy()
    ref = oracle.attention(qkv, arr["segment_ids"], plan.info["num_rows"], L, d, h)
    seg = arr["segment_ids"]
    for s_ in np.unique(seg[seg >= 0]):
        rows = seg == s_
        e = np.max(np.abs(got[rows] - ref[rows])) / np.max(np.abs(ref[rows]))
        assert e <= 2e-2, (s_, e)


def test_attention_bf16_long_runs_of_empty_query_blocks():
    """NaiveBatching layout (R17) with one 512-token request: every other row is a short
    request followed by ~490 pad slots, so most 128-slot query blocks are empty and each
    persistent CTA meets long runs of empty items between items with work (regression: the
    MMA issuer held the previous item's last P V back across them and deadlocked the Q ring).
    Per-request outputs vs the oracle on the First-Fit layout of the same requests (P4)."""
    rng = np.random.default_rng(23)
    n, d, h = 300, 256, 4
    lengths = np.concatenate([[512], rng.integers(3, 41, n - 1)]).astype(np.int32)
    T = int(lengths.sum())
    cu = np.concatenate([[0], np.cumsum(lengths)])
    tok = _bf16(rng.normal(size=(T, 3 * d)).astype(np.float32))

    def scatter(plan):
        a = plan.arrays()
        L = plan.info["row_len"]
        x = np.zeros((plan.num_slots, 3 * d), np.float32)
        for r in range(n):
            s0 = a["req_row"][r] * L + a["req_col"][r]
            x[s0:s0 + lengths[r]] = tok[cu[r]:cu[r + 1]]
        return a, x

    naive = tcb.tcb_pack(lengths, 512, 0, "naive")
    a_n, x_n = scatter(naive)
    out = tcb.op_attention(_dev(x_n, torch.bfloat16), _dev(a_n["segment_ids"]),
                           _dev(naive.segtab()), h)
    torch.cuda.synchronize()
    got = out.float().cpu().numpy()
    ff = tcb.tcb_pack(lengths, 512, 0)
    a_f, x_f = scatter(ff)
    ref = oracle.attention(x_f, a_f["segment_ids"], ff.info["num_rows"], 512, d, h)
    for r in range(n):
        g0 = a_n["req_row"][r] * 512 + a_n["req_col"][r]
        f0 = a_f["req_row"][r] * 512 + a_f["req_col"][r]
        g, o = got[g0:g0 + lengths[r]], ref[f0:f0 + lengths[r]]
        e = np.max(np.abs(g - o)) / np.max(np.abs(o))
        assert e <= 1.5e-2, (r, e)
    assert np.all(got[a_n["segment_ids"] < 0] == 0)


def test_attention_f32_vs_oracle():
    lengths = wl.draw_lengths("uniform_3_16", 8, 0)
    got, ref, seg = _attn_case(lengths, 32, 64, 2, "fp32", 2)
    assert np.max(np.abs(got - ref)) <= 2e-6


# ------------------------------------------------------------------- layernorm / embed --
@pytest.mark.parametrize("d", [512, 768, 1024])
def test_layernorm_bf16_vs_oracle(d):
    rng = np.random.default_rng(d)
    Z = _bf16(rng.normal(1.0, 3.0, size=(1031, d)))
    g = _bf16(1 + rng.normal(0, 0.1, size=d))
    b = _bf16(rng.normal(0, 0.1, size=d))
    seg = np.zeros(1031, np.int32)
    seg[-5:] = -1
    out = tcb.op_layernorm(_dev(Z, torch.bfloat16), _dev(g), _dev(b), 1e-5, _dev(seg))
    torch.cuda.synchronize()
    got = out.float().cpu().numpy()
    ref = oracle.layernorm(Z, g, b, 1e-5)
    assert np.all(np.abs(got[:-5] - ref[:-5]) <= 2.0 ** -8 * np.abs(ref[:-5]) + 2e-3)
    assert np.all(got[-5:] == 0)


def _scaled(mkey, pe, scale):
    import dataclasses
    m = wl.MODELS[mkey]
    return dataclasses.replace(m, name=f"{m.name}-{pe}-x{scale:g}", pe=pe, emb_scale=scale)


@pytest.mark.parametrize("mkey,L,pe,scale", [("toy", 32, None, None), ("transformer-base", 128, None, None),
                                             ("bert-base", 128, None, None),
                                             # ragged last 16-slot chunk of every row (40 = 2 x 16 + 8)
                                             ("toy", 40, None, None), ("bert-base", 40, None, None),
                                             # both sinusoidal readings (R1) with emb_scale != 1 (R3)
                                             ("transformer-base", 128, "sin_paper", 22.627416997969522),
                                             ("transformer-base", 128, "sin_vaswani", 2.5),
                                             ("toy", 32, "sin_vaswani", 8.0),
                                             # 64-slot chunks, slots in batches of 2 per warp:
                                             # ragged last chunk (104 = 64 + 40, 72 = 64 + 8)
                                             ("transformer-base", 104, None, None),
                                             ("bert-large", 72, None, None),
                                             ("transformer-big", 72, None, None)])
def test_pack_embed_metadata_bit_exact_and_values(mkey, L, pe, scale):
    model = wl.MODELS[mkey] if pe is None else _scaled(mkey, pe, scale)
    w = wl.draw_weights(model, 2)
    names = wl.weight_names(model)
    lengths = np.minimum(wl.draw_lengths("paracrawl", 90, 4), L).astype(np.int32)
    ids = wl.draw_token_ids(int(lengths.sum()), model.vocab, 5)
    enc = tcb.Encoder(model, w, names)
    plan = tcb.tcb_pack(lengths, L, 0)
    M = plan.num_slots
    segtab = _dev(plan.segtab())
    d_ids = _dev(ids)
    rows = enc.alloc_rows(M)
    seg = torch.full((M,), 7, dtype=torch.int32, device="cuda")
    pos = torch.full((M,), 7, dtype=torch.int32, device="cuda")
    enc.embed(plan, segtab, d_ids, rows, seg, pos)
    torch.cuda.synchronize()
    pk = oracle.pack(lengths, L)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L)
    assert seg.cpu().numpy().tolist() == lay["segment_ids"].tolist()
    assert pos.cpu().numpy().tolist() == lay["positions"].tolist()
    ref = oracle.embed(model, w, ids, lay)
    got = rows.float().cpu().numpy()
    tol = 1e-6 if model.dtype == "fp32" else 2.0 ** -8
    assert np.all(np.abs(got - ref) <= tol * np.abs(ref) + (1e-6 if model.dtype == "fp32" else 1e-3))


@pytest.mark.gpu
@pytest.mark.parametrize("dtype,d,L,lengths", [
    # fp32 d = 1024: 256 vectors per slot, a 16-slot chunk takes four load batches
    ("fp32", 1024, 40, [5, 17, 3, 30, 1, 8, 37, 2]),
    # bf16 d = 768, ragged last chunk of each row (40 = 2 x 16 + 8), pad slots
    ("bf16", 768, 40, [36, 1, 20, 20, 9, 4]),
    # row_len 4104: the row's segment records need > 48 KB of smem
    ("bf16", 64, 4104, [4104, 1, 4099, 7, 2000, 2000, 64] + [1] * 3100),
])
def test_unpack_exact_shapes(dtype, d, L, lengths):
    """a10: every request's tokens come back bit-exact and nothing else is written
    (sentinel-filled output), across load batches, ragged chunks and large row records."""
    model = small_model(dtype=dtype, d=d, h=d // 64, f=4 * d, max_pos=max(512, L))
    w = wl.draw_weights(model, 1)
    enc = tcb.Encoder(model, w, wl.weight_names(model))
    lengths = np.array(lengths, np.int32)
    plan = tcb.tcb_pack(lengths, L, 0)
    segtab = _dev(plan.segtab())
    tdt = torch.float32 if dtype == "fp32" else torch.bfloat16
    rows = torch.randn(plan.num_slots, d, device="cuda").to(tdt)
    T = int(lengths.sum())
    out = torch.full((T + 3, d), 12345.0, device="cuda").to(tdt)
    enc.unpack(plan, segtab, rows, out)
    torch.cuda.synchronize()
    a = plan.arrays()
    cu = np.concatenate([[0], np.cumsum(lengths)])
    r, o = rows.cpu(), out.cpu()
    for s, req in enumerate(a["seg_req"]):
        st = a["seg_start"][s]
        assert torch.equal(o[cu[req]:cu[req + 1]], r[st:st + lengths[req]])
    assert torch.all(o[T:] == 12345.0)


def test_unpack_roundtrip_exact():
    model = small_model(dtype="bf16", d=128, h=2, f=256)
    w = wl.draw_weights(model, 1)
    enc = tcb.Encoder(model, w, wl.weight_names(model))
    lengths = np.array([5, 17, 3, 30, 1, 8], np.int32)
    plan = tcb.tcb_pack(lengths, 32, 0, "first_fit_decreasing")
    segtab = _dev(plan.segtab())
    M = plan.num_slots
    rows = torch.randn(M, 128, device="cuda").to(torch.bfloat16)
    out = enc.unpack(plan, segtab, rows)
    torch.cuda.synchronize()
    a = plan.arrays()
    cu = np.concatenate([[0], np.cumsum(lengths)])
    r = rows.cpu()
    o = out.cpu()
    for s, req in enumerate(a["seg_req"]):
        st = a["seg_start"][s]
        assert torch.equal(o[cu[req]:cu[req + 1]], r[st:st + lengths[req]])


def test_attention_scheduler_variant_ops():
    """The scheduler-warp attention kernel (v3s; the forward uses it for rows of <= 128 slots)
    on every attention op test of this file: subprocess with TCB_ATTN_SCHED=1 (read once)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, TCB_ATTN_SCHED="1")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        "tests/test_gpu_kernels.py", "-k", "attention and not scheduler_variant"],
                       env=env, capture_output=True, text=True, cwd=root, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
