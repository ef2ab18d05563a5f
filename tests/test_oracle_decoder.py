"""Pins P14-P17 of the f4 decoder oracle (readings R30-R33, DESIGN.md §3/§4).

* P14: oracle_decoder_stack == torch.nn.TransformerDecoderLayer stack (post-LN, f64) with a
  causal tgt_mask and the request's own encoder output as memory.
* P15: greedy decoding: every step's logits == x_last . E_tok^T recomputed through torch's
  decoder on the oracle's own token prefix, and each token is the argmax (lowest index on
  ties) of its step's logits; decoding stops right after EOS.
* P16: causality -- decoder outputs at positions <= i do not depend on target tokens > i
  (bitwise), the property the GPU's incremental (KV-cache) decoding relies on.
* P17: the encoder half of a decode equals the packed encoder run (concat == alone, P4), so a
  request's decode does not depend on what it was batched with.
"""
import numpy as np
import torch

import oracle
import tcb_workload as wl


def _toy(act="relu", layers=2, d=64, h=2, f=256, vocab=97):
    return wl.ModelConfig("toy-dec", layers, d, h, f, vocab, 64, "fp32", act, "sin_paper", False,
                          False, 1e-5, 1e-5, 1.0)


def _torch_decoder(cfg, dw, x, mem):
    d, h = cfg.d_model, cfg.num_heads
    T = lambda a: torch.tensor(a, dtype=torch.float64)   # noqa: E731
    xt = T(x)[None]
    mt = T(mem)[None]
    t = x.shape[0]
    causal = torch.triu(torch.full((t, t), float("-inf"), dtype=torch.float64), diagonal=1)
    for layer in range(cfg.num_layers):
        m = torch.nn.TransformerDecoderLayer(d, h, cfg.d_ff, dropout=0.0, activation=cfg.act,
                                             layer_norm_eps=cfg.ln_eps, batch_first=True,
                                             norm_first=False, dtype=torch.float64)
        p = f"dec.l{layer}."
        with torch.no_grad():
            m.self_attn.in_proj_weight.copy_(T(dw[p + "w_qkv"]))
            m.self_attn.in_proj_bias.copy_(T(dw[p + "b_qkv"]))
            m.self_attn.out_proj.weight.copy_(T(dw[p + "w_o"]))
            m.self_attn.out_proj.bias.copy_(T(dw[p + "b_o"]))
            m.multihead_attn.in_proj_weight.copy_(T(np.concatenate([dw[p + "w_q"], dw[p + "w_kv"]])))
            m.multihead_attn.in_proj_bias.copy_(T(np.concatenate([dw[p + "b_q"], dw[p + "b_kv"]])))
            m.multihead_attn.out_proj.weight.copy_(T(dw[p + "w_co"]))
            m.multihead_attn.out_proj.bias.copy_(T(dw[p + "b_co"]))
            m.linear1.weight.copy_(T(dw[p + "w_1"]))
            m.linear1.bias.copy_(T(dw[p + "b_1"]))
            m.linear2.weight.copy_(T(dw[p + "w_2"]))
            m.linear2.bias.copy_(T(dw[p + "b_2"]))
            for k, ln in ((1, m.norm1), (2, m.norm2), (3, m.norm3)):
                ln.weight.copy_(T(dw[p + f"ln{k}_g"]))
                ln.bias.copy_(T(dw[p + f"ln{k}_b"]))
            xt = m(xt, mt, tgt_mask=causal)
    return xt[0].numpy()


def test_decoder_stack_vs_torch_transformer_decoder_layer():
    for act in ("relu", "gelu"):
        cfg = _toy(act)
        dw = wl.draw_dec_weights(cfg, 7)
        rng = np.random.default_rng(3)
        x = rng.normal(size=(11, cfg.d_model))
        mem = rng.normal(size=(9, cfg.d_model))
        got = oracle.decoder_stack(cfg, dw, wl.dec_weight_names(cfg), x, mem)
        ref = _torch_decoder(cfg, dw, x, mem)
        assert np.max(np.abs(got - ref)) <= 1e-12 * np.max(np.abs(ref)), act


def _embed_target(cfg, E, ys):
    d = cfg.d_model
    return np.array([[E[y, c] * cfg.emb_scale + oracle.pe(i, c, d, cfg.pe) for c in range(d)]
                     for i, y in enumerate(ys)])


def test_greedy_decode_logits_and_argmax_vs_torch():
    cfg = _toy()
    w = wl.draw_weights(cfg, 2)
    names = wl.weight_names(cfg)
    dw = wl.draw_dec_weights(cfg, 102)
    dn = wl.dec_weight_names(cfg)
    src = wl.draw_token_ids(8, cfg.vocab, 5)
    toks, lg = oracle.decode_greedy(cfg, w, names, dw, dn, src, 6, with_logits=True)
    assert len(toks) == 6 and lg.shape == (6, cfg.vocab)
    lay = oracle.layout([8], [0], [0], 1, 8)
    mem = oracle.encoder_rows(cfg, w, names, src, lay, 8)
    E = w["tok_emb"].astype(np.float64)
    ys = [wl.BOS]
    for k in range(len(toks)):
        x = _embed_target(cfg, E, ys)
        out = _torch_decoder(cfg, dw, x, mem)
        ref = out[-1] @ E.T
        assert np.max(np.abs(lg[k] - ref)) <= 1e-11 * np.max(np.abs(ref)), k
        top = np.flatnonzero(lg[k] == lg[k].max())
        assert toks[k] == top[0]                       # argmax, lowest index on ties
        ys.append(int(toks[k]))


def test_greedy_decode_eos_tmax_and_ties():
    """With the last LN3's gamma = 0 the decoder output is beta for every input, so the
    logits are beta . E_tok^T at every step: a row E[EOS] = 5 beta stops decoding after one
    token; without it, two identical best rows a < b tie and a must win at every one of the
    t_max steps."""
    cfg = _toy()
    w = dict(wl.draw_weights(cfg, 2))
    names, dn = wl.weight_names(cfg), wl.dec_weight_names(cfg)
    dw = dict(wl.draw_dec_weights(cfg, 102))
    last = f"dec.l{cfg.num_layers - 1}."
    beta = np.random.default_rng(8).normal(size=cfg.d_model).astype(np.float32)
    dw[last + "ln3_g"] = np.zeros(cfg.d_model, np.float32)
    dw[last + "ln3_b"] = beta
    src = wl.draw_token_ids(8, cfg.vocab, 5)
    E = w["tok_emb"].copy()
    E[wl.EOS] = 5.0 * beta
    w["tok_emb"] = E
    toks = oracle.decode_greedy(cfg, w, names, dw, dn, src, 6)
    assert list(toks) == [wl.EOS]
    E = wl.draw_weights(cfg, 2)["tok_emb"].copy()
    a, b = 40, 71
    E[a] = E[b] = 4.0 * beta
    w["tok_emb"] = E
    toks, lg = oracle.decode_greedy(cfg, w, names, dw, dn, src, 6, with_logits=True)
    assert list(toks) == [a] * 6
    assert np.all(lg[:, a] == lg[:, b])


def test_decoder_causality_bitwise():
    cfg = _toy()
    dw = wl.draw_dec_weights(cfg, 9)
    rng = np.random.default_rng(4)
    x = rng.normal(size=(10, cfg.d_model))
    mem = rng.normal(size=(7, cfg.d_model))
    a = oracle.decoder_stack(cfg, dw, wl.dec_weight_names(cfg), x, mem)
    x2 = x.copy()
    x2[6:] = rng.normal(size=(4, cfg.d_model))
    b = oracle.decoder_stack(cfg, dw, wl.dec_weight_names(cfg), x2, mem)
    assert np.array_equal(a[:6], b[:6])
    assert not np.array_equal(a[6:], b[6:])
    # the prefix alone gives the same rows (what an incremental decoder computes)
    c = oracle.decoder_stack(cfg, dw, wl.dec_weight_names(cfg), x[:6], mem)
    assert np.array_equal(a[:6], c)


def test_decode_memory_is_the_packed_encoder_output():
    cfg = _toy()
    w = wl.draw_weights(cfg, 2)
    names = wl.weight_names(cfg)
    lengths = np.array([8, 5, 11], np.int32)
    ids = wl.draw_token_ids(int(lengths.sum()), cfg.vocab, 6)
    packed = oracle.run(cfg, w, names, lengths, ids, 32)["out"]
    cu = np.concatenate([[0], np.cumsum(lengths)])
    for r, l in enumerate(lengths):
        lay = oracle.layout([l], [0], [0], 1, int(l))
        alone = oracle.encoder_rows(cfg, w, names, ids[cu[r]:cu[r + 1]], lay, int(l))
        assert np.array_equal(alone, packed[cu[r]:cu[r + 1]])
