"""Pins P3, P5, P6, P8 of the oracle's arithmetic -- DESIGN.md §4.

* P3: Eq. (1)-(2) sinusoidal PE, closed form at hand-evaluated points
  (tests/golden/f1_layout.json) and the special case PE(0, .) = [0, 1, 0, 1, ...].
* P5: one request filling a whole row with no padding -> textbook scaled-dot-product
  attention (Eq. (4)) == torch.nn.functional.scaled_dot_product_attention.
* P6: the oracle's S-layer stack == torch.nn.TransformerEncoderLayer (post-LN, f64) with a
  block-diagonal src_mask (Eq. (5)-(6)), on the oracle's embedded X.
* P8: identities -- LayerNorm output statistics, GELU(0) = 0, ReLU, linear with identity.
"""
import json
import math
import os

import numpy as np
import pytest
import torch

import oracle
import tcb_workload as wl


def test_pe_closed_form_golden(golden_dir):
    f1 = json.load(open(os.path.join(golden_dir, "f1_layout.json")))
    got = [oracle.pe(1, c, 64, "sin_paper") for c in range(4)]
    assert np.allclose(got, f1["pe_pos1_d64_dims0to3_sin_paper"], rtol=0, atol=2e-16)
    got = [oracle.pe(1, c, 64, "sin_vaswani") for c in range(4)]
    assert np.allclose(got, f1["pe_pos1_d64_dims0to3_sin_vaswani"], rtol=0, atol=2e-16)
    # R1 is observable: the two variants differ first at dim 1
    assert oracle.pe(1, 1, 64, "sin_paper") != oracle.pe(1, 1, 64, "sin_vaswani")


def test_pe_origin_and_large_dims():
    for d in (64, 512):
        row = [oracle.pe(0, c, d, "sin_paper") for c in range(d)]
        assert row == [0.0 if c % 2 == 0 else 1.0 for c in range(d)]
    # highest even dim: sin(pos / 10000^((d-2)/d))
    assert oracle.pe(7, 510, 512) == pytest.approx(math.sin(7 / 10000 ** (510 / 512)), abs=1e-15)


def _toy_inputs(seed=5, d=64, h=2, f=256, layers=2, act="gelu"):
    cfg = wl.ModelConfig("t", layers, d, h, f, 50, 64, "fp32", act, "sin_paper", False, False,
                         1e-5, 1e-5, 1.0)
    w = wl.draw_weights(cfg, seed)
    return cfg, w


def test_sdpa_special_case_single_full_row():
    """P5: a row holding exactly one request -> the mask is all zeros -> Eq. (4)."""
    rng = np.random.default_rng(7)
    L, d, h = 24, 64, 4
    qkv = rng.normal(size=(L, 3 * d))
    seg = np.zeros(L, np.int32)
    o = oracle.attention(qkv, seg, 1, L, d, h)
    t = torch.tensor(qkv, dtype=torch.float64)
    q, k, v = t[:, :d], t[:, d:2 * d], t[:, 2 * d:]
    sh = lambda x: x.view(L, h, d // h).transpose(0, 1)   # noqa: E731
    ref = torch.nn.functional.scaled_dot_product_attention(sh(q), sh(k), sh(v))
    ref = ref.transpose(0, 1).reshape(L, d).numpy()
    assert np.max(np.abs(o - ref)) <= 1e-13 * np.max(np.abs(ref))


def test_masked_attention_equals_per_segment_sdpa():
    """Eq. (5)-(7): with the block mask, each segment's rows equal SDPA on that segment."""
    rng = np.random.default_rng(8)
    L, d, h = 40, 32, 2
    seg = np.array([0] * 11 + [1] * 5 + [2] * 20 + [-1] * 4, np.int32)
    qkv = rng.normal(size=(L, 3 * d))
    o = oracle.attention(qkv, seg, 1, L, d, h)
    t = torch.tensor(qkv, dtype=torch.float64)
    for s, (a, b) in enumerate([(0, 11), (11, 16), (16, 36)]):
        q, k, v = t[a:b, :d], t[a:b, d:2 * d], t[a:b, 2 * d:]
        sh = lambda x: x.reshape(b - a, h, d // h).transpose(0, 1)   # noqa: E731
        ref = torch.nn.functional.scaled_dot_product_attention(sh(q), sh(k), sh(v))
        ref = ref.transpose(0, 1).reshape(b - a, d).numpy()
        assert np.max(np.abs(o[a:b] - ref)) <= 1e-13
    assert (o[36:] == 0).all()   # pad queries (R12)


def _torch_layers(cfg, w, x, seg, L):
    """torch.nn.TransformerEncoderLayer stack, f64, batch_first, post-LN, block mask."""
    B = x.shape[0] // L
    d, h = cfg.d_model, cfg.num_heads
    xs = torch.tensor(x.reshape(B, L, d), dtype=torch.float64)
    seg = seg.reshape(B, L)
    mask = torch.full((B, L, L), float("-inf"), dtype=torch.float64)
    for b in range(B):
        for i in range(L):
            for j in range(L):
                if (seg[b, i] >= 0 and seg[b, i] == seg[b, j]) or (seg[b, i] < 0 and i == j):
                    mask[b, i, j] = 0.0
    mask = mask.repeat_interleave(h, dim=0)   # (B*h, L, L), batch-major as torch expects
    for layer in range(cfg.num_layers):
        m = torch.nn.TransformerEncoderLayer(d, h, cfg.d_ff, dropout=0.0, activation=cfg.act,
                                             layer_norm_eps=cfg.ln_eps, batch_first=True,
                                             norm_first=False, dtype=torch.float64)
        p = f"l{layer}."
        T = lambda a: torch.tensor(a, dtype=torch.float64)   # noqa: E731
        with torch.no_grad():
            m.self_attn.in_proj_weight.copy_(T(w[p + "w_qkv"]))
            m.self_attn.in_proj_bias.copy_(T(w[p + "b_qkv"]))
            m.self_attn.out_proj.weight.copy_(T(w[p + "w_o"]))
            m.self_attn.out_proj.bias.copy_(T(w[p + "b_o"]))
            m.norm1.weight.copy_(T(w[p + "ln1_g"]))
            m.norm1.bias.copy_(T(w[p + "ln1_b"]))
            m.linear1.weight.copy_(T(w[p + "w_1"]))
            m.linear1.bias.copy_(T(w[p + "b_1"]))
            m.linear2.weight.copy_(T(w[p + "w_2"]))
            m.linear2.bias.copy_(T(w[p + "b_2"]))
            m.norm2.weight.copy_(T(w[p + "ln2_g"]))
            m.norm2.bias.copy_(T(w[p + "ln2_b"]))
        m.eval()
        with torch.no_grad():
            xs = m(xs, src_mask=mask)
    return xs.reshape(B * L, d).numpy()


@pytest.mark.parametrize("act", ["gelu", "relu"])
def test_encoder_stack_equals_torch_transformer_layer(act):
    """P6: o3-o7 against torch's own encoder layer, f64, on the oracle's embedded X."""
    cfg, w = _toy_inputs(act=act)
    names = wl.weight_names(cfg)
    lengths = np.array([9, 7, 12, 3, 5, 16, 4], np.int32)
    L = 24
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 3)
    pk = oracle.pack(lengths, L)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L)
    x0 = oracle.embed(cfg, w, ids, lay)
    got = oracle.encoder_rows(cfg, w, names, ids, lay, L)
    ref = _torch_layers(cfg, w, x0, lay["segment_ids"], L)
    real = lay["segment_ids"] >= 0
    err = np.max(np.abs(got[real] - ref[real])) / np.max(np.abs(ref[real]))
    assert err <= 1e-12, err
    assert (got[~real] == 0).all()


def test_bert_embedding_against_transformers_style_reference():
    """Embedding with learned restarted positions + type-0 + LN_emb (R4, R5): written out
    directly with torch ops (E[id] + P[pos] + T0, LayerNorm) on the layout's positions."""
    cfg = wl.ModelConfig("b", 1, 64, 2, 256, 100, 64, "fp32", "gelu", "learned", True, True,
                         1e-12, 1e-12, 1.0)
    w = wl.draw_weights(cfg, 9)
    lengths = np.array([10, 20, 5], np.int32)
    L = 32
    ids = wl.draw_token_ids(35, cfg.vocab, 4)
    pk = oracle.pack(lengths, L)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L)
    x = oracle.embed(cfg, w, ids, lay)
    T = lambda a: torch.tensor(a, dtype=torch.float64)   # noqa: E731
    for s in np.nonzero(lay["segment_ids"] >= 0)[0]:
        e = T(w["tok_emb"][ids[lay["tok_index"][s]]]) + T(w["pos_emb"][lay["positions"][s]]) \
            + T(w["type_emb"])
        ref = torch.nn.functional.layer_norm(e, (64,), T(w["emb_ln_g"]), T(w["emb_ln_b"]), 1e-12)
        assert np.max(np.abs(x[s] - ref.numpy())) < 1e-13


def test_identities():
    """P8."""
    rng = np.random.default_rng(11)
    z = rng.normal(3.0, 2.0, size=(5, 128))
    y = oracle.layernorm(z, np.ones(128), np.zeros(128), 0.0)
    assert np.max(np.abs(y.mean(1))) < 1e-14
    assert np.max(np.abs(y.var(1) - 1.0)) < 1e-13
    x = rng.normal(size=(3, 16))
    eye = np.eye(16)
    assert np.array_equal(oracle.linear(x, eye, np.zeros(16)), x)
    assert np.array_equal(oracle.linear(x, eye, np.zeros(16), act="relu"), np.maximum(x, 0))
    g = oracle.linear(np.zeros((1, 4)), np.eye(4), np.zeros(4), act="gelu")
    assert (g == 0).all()
    # GELU(u) against the erf closed form at a few points
    u = np.array([[-3.0, -1.0, 0.5, 2.0]])
    g = oracle.linear(u, np.eye(4), np.zeros(4), act="gelu")
    ref = [0.5 * v * (1 + math.erf(v / math.sqrt(2))) for v in u[0]]
    assert np.allclose(g[0], ref, rtol=0, atol=1e-16)
    # softmax rows sum to one: attention with V = ones gives ones
    L, d = 10, 8
    qkv = rng.normal(size=(L, 3 * d))
    qkv[:, 2 * d:] = 1.0
    o = oracle.attention(qkv, np.array([0] * 6 + [1] * 4, np.int32), 1, L, d, 1)
    assert np.max(np.abs(o - 1.0)) <= 4 * np.finfo(float).eps


@pytest.mark.parametrize("pe,scale", [("sin_paper", 1.0), ("sin_paper", 2.5),
                                      ("sin_vaswani", 8.0), ("sin_vaswani", 1.0)])
def test_sinusoidal_embedding_closed_form(pe, scale):
    """oracle_embed's sinusoidal branch (Eq. (1)-(2) P:329-333, separate PE §4.1.1)
    against the closed form written out here: x = E[id] * emb_scale + PE(j, c) with j the
    token's index inside its own request (positions restart, R2), PE(j, c) = sin / cos of
    j / 10000^(c/d) for the literal Eq. (2) (R1: odd columns use (2e+1)/d) or of
    j / 10000^(2 floor(c/2)/d) (Vaswani), every slot located from the packing alone
    (row * L + col + j); pad slots are 0."""
    d = 64
    cfg = wl.ModelConfig("s", 1, d, 2, 256, 100, 64, "fp32", "relu", pe, False, False,
                         1e-5, 1e-5, scale)
    w = wl.draw_weights(cfg, 5)
    lengths = np.array([7, 12, 3, 9, 16, 5], np.int32)
    L = 24
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 6)
    pk = oracle.pack(lengths, L)
    lay = oracle.layout(lengths, pk["req_row"], pk["req_col"], pk["num_rows"], L)
    x = oracle.embed(cfg, w, ids, lay)
    cu = np.concatenate([[0], np.cumsum(lengths)])
    real = np.zeros(len(x), bool)
    for r, l in enumerate(lengths):
        for j in range(l):
            slot = pk["req_row"][r] * L + pk["req_col"][r] + j
            real[slot] = True
            ref = np.array(w["tok_emb"][ids[cu[r] + j]], np.float64) * scale
            for c in range(d):
                ex = c / d if pe == "sin_paper" else (c - c % 2) / d
                ang = j / 10000.0 ** ex
                ref[c] += math.sin(ang) if c % 2 == 0 else math.cos(ang)
            assert np.max(np.abs(x[slot] - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref))), (r, j)
    assert np.all(x[~real] == 0)
