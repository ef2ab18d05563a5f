"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This module holds NO arithmetic of the method (no packing, no embedding, no attention,
no layer math).  It only draws numbers: request lengths, token ids and random-init
weights, with the shapes and distributions of SURVEY.md §8(d) / DESIGN.md §"Input recipe".
Both sides (``oracle/`` and the CUDA path) consume exactly the arrays produced here.

Paper context (PAPER.md = /root/reference/PAPER.md, not read at run time):
  * requests are sentences of l_n tokens (§5.1 "Problem statement"),
  * the paper's own stream draws lengths 3-100 from a normal distribution with mean 20
    and variance 20 / 100 (§6.2) -> ``paper_normal`` below (reading R19),
  * model dims come from BASELINE.json ``configs`` (reading R20: the paper's d_model=3072
    is not used).
"""
from __future__ import annotations

import dataclasses
from typing import Dict, List

import numpy as np


@dataclasses.dataclass(frozen=True)
class ModelConfig:
    """Encoder hyper-parameters (BASELINE.json configs; readings R3-R10 in DESIGN.md)."""

    name: str
    num_layers: int
    d_model: int
    num_heads: int
    d_ff: int
    vocab: int
    max_pos: int
    dtype: str          # "fp32" | "bf16"  (storage/compute dtype of the CUDA path)
    act: str            # "gelu" (erf form) | "relu"            (reading R9)
    pe: str             # "sin_paper" | "sin_vaswani" | "learned" (readings R1, R4)
    emb_ln: bool        # BERT embedding LayerNorm              (reading R5)
    use_type_emb: bool  # BERT token-type-0 embedding           (reading R5)
    ln_eps: float       # (reading R10)
    emb_ln_eps: float
    emb_scale: float    # (reading R3)

    @property
    def d_head(self) -> int:
        return self.d_model // self.num_heads


@dataclasses.dataclass(frozen=True)
class Workload:
    """One BASELINE.json config: a model, a row shape and a length distribution."""

    name: str
    model: ModelConfig
    row_len: int        # L  (every batch is B rows x L words)
    rows: int           # B per GPU
    lengths: str        # name of the length distribution
    seeds: tuple        # (lengths seed, ids seed, weights seed)


MODELS: Dict[str, ModelConfig] = {
    "toy": ModelConfig("toy", 2, 64, 2, 256, 128, 64, "fp32", "gelu", "sin_paper",
                       False, False, 1e-5, 1e-5, 1.0),
    "transformer-base": ModelConfig("transformer-base", 6, 512, 8, 2048, 32000, 512, "bf16",
                                    "relu", "sin_paper", False, False, 1e-5, 1e-5, 1.0),
    "bert-base": ModelConfig("bert-base", 12, 768, 12, 3072, 30522, 512, "bf16", "gelu",
                             "learned", True, True, 1e-12, 1e-12, 1.0),
    "bert-large": ModelConfig("bert-large", 24, 1024, 16, 4096, 30522, 512, "bf16", "gelu",
                              "learned", True, True, 1e-12, 1e-12, 1.0),
    "transformer-big": ModelConfig("transformer-big", 6, 1024, 16, 4096, 32000, 512, "bf16",
                                   "relu", "sin_paper", False, False, 1e-5, 1e-5, 1.0),
}

WORKLOADS: Dict[str, Workload] = {
    "c1": Workload("c1-toy", MODELS["toy"], 32, 2, "uniform_3_16", (0, 1, 2)),
    "c2": Workload("c2-transformer-base-paracrawl", MODELS["transformer-base"], 128, 256,
                   "paracrawl", (10, 11, 12)),
    "c3": Workload("c3-bert-base-dia", MODELS["bert-base"], 512, 64, "dia", (20, 21, 22)),
    "c4": Workload("c4-bert-large-mixed", MODELS["bert-large"], 512, 64, "mixed_8_512",
                   (30, 31, 32)),
    "c5": Workload("c5-transformer-big-wmt", MODELS["transformer-big"], 256, 128, "wmt",
                   (40, 41, 42)),
}


# ----------------------------------------------------------------------------------------
# Length distributions (SURVEY.md §8(d) table "Synthetic inputs")
# ----------------------------------------------------------------------------------------
def draw_lengths(dist: str, n: int, seed: int) -> np.ndarray:
    """Draw ``n`` request lengths (int32) from a named distribution with ``seed``."""
    rng = np.random.default_rng(seed)
    if dist == "uniform_3_16":            # C1 toy
        x = rng.integers(3, 17, size=n)
    elif dist == "paracrawl":             # C2: round(LogNormal(ln 24, 0.7)) clip [2, 128]
        x = np.clip(np.rint(rng.lognormal(np.log(24.0), 0.7, size=n)), 2, 128)
    elif dist == "dia":                   # C3: 60% LogNormal(ln 32, .6) clip [8,512]; 40% U[128,512]
        a = np.clip(np.rint(rng.lognormal(np.log(32.0), 0.6, size=n)), 8, 512)
        b = rng.integers(128, 513, size=n)
        pick = rng.random(size=n) < 0.6
        x = np.where(pick, a, b)
    elif dist == "mixed_8_512":           # C4: round(exp(U(ln 8, ln 512)))
        x = np.rint(np.exp(rng.uniform(np.log(8.0), np.log(512.0), size=n)))
    elif dist == "wmt":                   # C5: round(LogNormal(ln 26, .55)) clip [3, 256]
        x = np.clip(np.rint(rng.lognormal(np.log(26.0), 0.55, size=n)), 3, 256)
    elif dist == "paper_normal_20":       # PAPER.md:1539-1541, variance 20 (R19)
        x = np.clip(np.rint(rng.normal(20.0, np.sqrt(20.0), size=n)), 3, 100)
    elif dist == "paper_normal_100":      # PAPER.md:1647-1650, variance 100 (R19)
        x = np.clip(np.rint(rng.normal(20.0, np.sqrt(100.0), size=n)), 3, 100)
    else:
        raise ValueError(f"unknown length distribution {dist!r}")
    return np.ascontiguousarray(x.astype(np.int32))


def lengths_filling(dist: str, rows: int, row_len: int, seed: int,
                    fill: float = 0.995) -> np.ndarray:
    """Draw a stream prefix whose total tokens is about ``fill * rows * row_len``.

    The stream is the first k requests of an infinite seeded stream (chunks of 4096 are
    drawn with seeds seed, seed+1, ...), so the result is deterministic.  The caller packs
    it; with max_rows=rows a First-Fit packer places (almost) all of it.
    """
    target = int(fill * rows * row_len)
    out: List[np.ndarray] = []
    total = 0
    chunk = 0
    while total < target:
        x = draw_lengths(dist, 4096, seed + 7919 * chunk)
        chunk += 1
        cs = np.cumsum(x)
        k = int(np.searchsorted(cs, target - total, side="right"))
        out.append(x[:k])
        total += int(cs[k - 1]) if k > 0 else 0
        if k < len(x):
            break
    return np.ascontiguousarray(np.concatenate(out).astype(np.int32))


def draw_token_ids(total_tokens: int, vocab: int, seed: int) -> np.ndarray:
    """Token ids uniform in [0, vocab), request order, int32 (reading R24)."""
    rng = np.random.default_rng(seed)
    return np.ascontiguousarray(rng.integers(0, vocab, size=total_tokens).astype(np.int32))


# ----------------------------------------------------------------------------------------
# Weights (reading R22: drawn in fp32, rounded once to bf16 with RNE for bf16 models)
# ----------------------------------------------------------------------------------------
GLOBAL_WEIGHT_NAMES = ["tok_emb", "pos_emb", "type_emb", "emb_ln_g", "emb_ln_b"]
LAYER_WEIGHT_NAMES = ["w_qkv", "b_qkv", "w_o", "b_o", "ln1_g", "ln1_b",
                      "w_1", "b_1", "w_2", "b_2", "ln2_g", "ln2_b"]


def weight_names(cfg: ModelConfig) -> List[str]:
    names = list(GLOBAL_WEIGHT_NAMES)
    for layer in range(cfg.num_layers):
        names += [f"l{layer}.{n}" for n in LAYER_WEIGHT_NAMES]
    return names


def weight_shapes(cfg: ModelConfig) -> Dict[str, tuple]:
    d, f = cfg.d_model, cfg.d_ff
    shapes = {
        "tok_emb": (cfg.vocab, d),
        "pos_emb": (cfg.max_pos if cfg.pe == "learned" else 1, d),
        "type_emb": (d,),
        "emb_ln_g": (d,),
        "emb_ln_b": (d,),
    }
    per = {"w_qkv": (3 * d, d), "b_qkv": (3 * d,), "w_o": (d, d), "b_o": (d,),
           "ln1_g": (d,), "ln1_b": (d,), "w_1": (f, d), "b_1": (f,), "w_2": (d, f),
           "b_2": (d,), "ln2_g": (d,), "ln2_b": (d,)}
    for layer in range(cfg.num_layers):
        for n, s in per.items():
            shapes[f"l{layer}.{n}"] = s
    return shapes


def round_to_bf16(x: np.ndarray) -> np.ndarray:
    """Round fp32 values to the nearest bf16 (ties to even); returns fp32 holding them."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    u = (u + 0x7FFF + lsb) >> 16 << 16
    return (u.astype(np.uint32)).view(np.float32).copy()


def bf16_bits(x: np.ndarray) -> np.ndarray:
    """The uint16 bf16 bit patterns of values already representable in bf16."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    return (x.view(np.uint32) >> 16).astype(np.uint16)


def draw_weights(cfg: ModelConfig, seed: int) -> Dict[str, np.ndarray]:
    """Random-init weights (SURVEY.md §8(d) "Weights"), fp32 arrays in canonical order."""
    rng = np.random.default_rng(seed)
    shapes = weight_shapes(cfg)
    d = cfg.d_model
    out: Dict[str, np.ndarray] = {}
    for name in weight_names(cfg):
        shp = shapes[name]
        base = name.split(".")[-1]
        if base in ("w_qkv", "w_o", "w_1", "w_2"):
            fan_out, fan_in = shp
            if base == "w_qkv":
                fan_out = d           # xavier per projection, as torch in_proj does
            a = np.sqrt(6.0 / (fan_in + fan_out))
            w = rng.uniform(-a, a, size=shp)
        elif base.startswith("b_"):
            w = rng.normal(0.0, 0.02, size=shp)
        elif base.endswith("_g"):
            w = 1.0 + rng.normal(0.0, 0.1, size=shp)
        elif base.endswith("_b"):
            w = rng.normal(0.0, 0.1, size=shp)
        elif base == "tok_emb":
            w = rng.normal(0.0, 1.0, size=shp)
        elif base in ("pos_emb", "type_emb"):
            w = rng.normal(0.0, 0.02, size=shp)
        else:  # pragma: no cover
            raise AssertionError(name)
        w = w.astype(np.float32)
        if cfg.dtype == "bf16":
            w = round_to_bf16(w)
        out[name] = np.ascontiguousarray(w)
    return out


def workload_inputs(key: str, rows: int | None = None, fill: float = 0.995):
    """(lengths, token_ids, weights) for a WORKLOADS key, sized for ``rows`` rows."""
    wl = WORKLOADS[key]
    rows = wl.rows if rows is None else rows
    if key == "c1":
        lengths = draw_lengths(wl.lengths, 8, wl.seeds[0])
    else:
        lengths = lengths_filling(wl.lengths, rows, wl.row_len, wl.seeds[0], fill)
    ids = draw_token_ids(int(lengths.sum()), wl.model.vocab, wl.seeds[1])
    weights = draw_weights(wl.model, wl.seeds[2])
    return lengths, ids, weights


# ----------------------------------------------------------------------------------------
# f4: the decoder of the Seq2Seq setting (readings R30-R33 in DESIGN.md)
# ----------------------------------------------------------------------------------------
BOS, EOS = 1, 2                      # reading R31
DEC_LAYER_WEIGHT_NAMES = ["w_qkv", "b_qkv", "w_o", "b_o", "ln1_g", "ln1_b",
                          "w_q", "b_q", "w_kv", "b_kv", "w_co", "b_co", "ln2_g", "ln2_b",
                          "w_1", "b_1", "w_2", "b_2", "ln3_g", "ln3_b"]


def dec_weight_names(cfg: ModelConfig) -> List[str]:
    return [f"dec.l{layer}.{n}" for layer in range(cfg.num_layers) for n in DEC_LAYER_WEIGHT_NAMES]


def max_target_len(l_src: int, cfg: ModelConfig) -> int:
    """Reading R32: a request may generate up to as many tokens as its source has (a
    translation-like budget), capped so every target position has a PE row."""
    return int(min(l_src, cfg.max_pos - 1))


def draw_dec_weights(cfg: ModelConfig, seed: int) -> Dict[str, np.ndarray]:
    """Random-init decoder weights with the encoder's recipe (Xavier linears, N(0, .02^2)
    biases, LN gamma 1 + N(0, .1^2), beta N(0, .1^2)); rounded to bf16 for bf16 models."""
    rng = np.random.default_rng(seed)
    d, f = cfg.d_model, cfg.d_ff
    shapes = {"w_qkv": (3 * d, d), "b_qkv": (3 * d,), "w_o": (d, d), "b_o": (d,),
              "ln1_g": (d,), "ln1_b": (d,), "w_q": (d, d), "b_q": (d,), "w_kv": (2 * d, d),
              "b_kv": (2 * d,), "w_co": (d, d), "b_co": (d,), "ln2_g": (d,), "ln2_b": (d,),
              "w_1": (f, d), "b_1": (f,), "w_2": (d, f), "b_2": (d,), "ln3_g": (d,),
              "ln3_b": (d,)}
    out: Dict[str, np.ndarray] = {}
    for name in dec_weight_names(cfg):
        base = name.split(".")[-1]
        shp = shapes[base]
        if base.startswith("w_"):
            fan_out, fan_in = shp
            if base in ("w_qkv", "w_kv"):
                fan_out = d           # per projection, as torch's in_proj
            a = np.sqrt(6.0 / (fan_in + fan_out))
            w = rng.uniform(-a, a, size=shp)
        elif base.startswith("b_"):
            w = rng.normal(0.0, 0.02, size=shp)
        elif base.endswith("_g"):
            w = 1.0 + rng.normal(0.0, 0.1, size=shp)
        else:
            w = rng.normal(0.0, 0.1, size=shp)
        w = w.astype(np.float32)
        if cfg.dtype == "bf16":
            w = round_to_bf16(w)
        out[name] = np.ascontiguousarray(w)
    return out
