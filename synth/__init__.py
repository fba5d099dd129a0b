"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no forward pass, no planner, no
simulator).  It only draws data:

* model shape descriptions of the paper's models (PAPER.md P:241 names BERT-Base/
  Large, RoBERTa-Base/Large, GPT-2 / GPT-2 Medium from HF Transformers [35]; the
  shapes are the standard HF configs -- SURVEY §8 table);
* random-init weights in HF state-dict naming;
* token ids (the paper uses "a synthetic dataset");
* random integer cost tables for planner tests;
* seeded Poisson request traces for the serving harness.

Every generator is numpy PCG64 with a fixed seed.  Both the oracle (tests only)
and the product path (through the C-ABI) consume the same arrays; neither side
imports the other.
"""
from __future__ import annotations

import dataclasses
from collections import OrderedDict

import numpy as np

# --------------------------------------------------------------------------------------
# Model shapes (HF configs).  family: "bert" | "roberta" | "gpt2"
# --------------------------------------------------------------------------------------


@dataclasses.dataclass(frozen=True)
class ModelShape:
    name: str
    family: str
    vocab: int
    max_pos: int
    type_vocab: int
    hidden: int
    heads: int
    ffn: int
    layers: int
    ln_eps: float
    pad_idx: int = 0  # roberta: 1 (position ids start at pad_idx+1)


SHAPES = {
    # tiny BERT: BASELINE.json configs[0]; ffn/max_pos/type_vocab proposed
    "tiny_bert": ModelShape("tiny_bert", "bert", 1000, 512, 2, 128, 2, 512, 2, 1e-12),
    "bert_base": ModelShape("bert_base", "bert", 30522, 512, 2, 768, 12, 3072, 12, 1e-12),
    "bert_large": ModelShape("bert_large", "bert", 30522, 512, 2, 1024, 16, 4096, 24, 1e-12),
    "roberta_base": ModelShape("roberta_base", "roberta", 50265, 514, 1, 768, 12, 3072, 12, 1e-5, 1),
    "roberta_large": ModelShape("roberta_large", "roberta", 50265, 514, 1, 1024, 16, 4096, 24, 1e-5, 1),
    "gpt2": ModelShape("gpt2", "gpt2", 50257, 1024, 0, 768, 12, 3072, 12, 1e-5),
    "gpt2_medium": ModelShape("gpt2_medium", "gpt2", 50257, 1024, 0, 1024, 16, 4096, 24, 1e-5),
    # small test shapes (several tiles + ragged tails; not paper models)
    "tiny_roberta": ModelShape("tiny_roberta", "roberta", 1000, 130, 1, 128, 2, 512, 2, 1e-5, 1),
    "tiny_gpt2": ModelShape("tiny_gpt2", "gpt2", 1000, 256, 0, 128, 2, 512, 2, 1e-5),
}


def hf_param_shapes(m: ModelShape) -> "OrderedDict[str, tuple]":
    """HF state-dict names and shapes, in HF forward (registration) order."""
    H, F = m.hidden, m.ffn
    out: "OrderedDict[str, tuple]" = OrderedDict()
    if m.family in ("bert", "roberta"):
        out["embeddings.word_embeddings.weight"] = (m.vocab, H)
        out["embeddings.position_embeddings.weight"] = (m.max_pos, H)
        out["embeddings.token_type_embeddings.weight"] = (m.type_vocab, H)
        out["embeddings.LayerNorm.weight"] = (H,)
        out["embeddings.LayerNorm.bias"] = (H,)
        for i in range(m.layers):
            p = f"encoder.layer.{i}."
            for nm in ("query", "key", "value"):
                out[p + f"attention.self.{nm}.weight"] = (H, H)
                out[p + f"attention.self.{nm}.bias"] = (H,)
            out[p + "attention.output.dense.weight"] = (H, H)
            out[p + "attention.output.dense.bias"] = (H,)
            out[p + "attention.output.LayerNorm.weight"] = (H,)
            out[p + "attention.output.LayerNorm.bias"] = (H,)
            out[p + "intermediate.dense.weight"] = (F, H)
            out[p + "intermediate.dense.bias"] = (F,)
            out[p + "output.dense.weight"] = (H, F)
            out[p + "output.dense.bias"] = (H,)
            out[p + "output.LayerNorm.weight"] = (H,)
            out[p + "output.LayerNorm.bias"] = (H,)
        out["pooler.dense.weight"] = (H, H)
        out["pooler.dense.bias"] = (H,)
    elif m.family == "gpt2":
        out["wte.weight"] = (m.vocab, H)
        out["wpe.weight"] = (m.max_pos, H)
        for i in range(m.layers):
            p = f"h.{i}."
            out[p + "ln_1.weight"] = (H,)
            out[p + "ln_1.bias"] = (H,)
            out[p + "attn.c_attn.weight"] = (H, 3 * H)  # Conv1D: [in, out]
            out[p + "attn.c_attn.bias"] = (3 * H,)
            out[p + "attn.c_proj.weight"] = (H, H)
            out[p + "attn.c_proj.bias"] = (H,)
            out[p + "ln_2.weight"] = (H,)
            out[p + "ln_2.bias"] = (H,)
            out[p + "mlp.c_fc.weight"] = (H, F)
            out[p + "mlp.c_fc.bias"] = (F,)
            out[p + "mlp.c_proj.weight"] = (F, H)
            out[p + "mlp.c_proj.bias"] = (H,)
        out["ln_f.weight"] = (H,)
        out["ln_f.bias"] = (H,)
    else:
        raise ValueError(m.family)
    return out


# --------------------------------------------------------------------------------------
# Rounding to the storage dtype (round-to-nearest-even)
# --------------------------------------------------------------------------------------

def to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 bit patterns (uint16), round-to-nearest-even (finite inputs)."""
    u = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32)
    rounding = ((u >> 16) & 1) + np.uint32(0x7FFF)
    return ((u + rounding) >> 16).astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (b.astype(np.uint32) << 16).view(np.float32)


def round_to(x: np.ndarray, dtype: str) -> np.ndarray:
    """Round fp32 data to the storage dtype; returns the storage array.

    fp16 -> np.float16 (numpy astype is RNE); bf16 -> np.uint16 bit patterns;
    fp32 -> np.float32.
    """
    if dtype == "fp16":
        return np.asarray(x, dtype=np.float32).astype(np.float16)
    if dtype == "bf16":
        return to_bf16_bits(x)
    if dtype == "fp32":
        return np.asarray(x, dtype=np.float32)
    raise ValueError(dtype)


def storage_to_f64(a: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "bf16":
        return bf16_bits_to_f32(a).astype(np.float64)
    return a.astype(np.float64)


# --------------------------------------------------------------------------------------
# Weights: matrices/embeddings/biases ~ N(0, std^2);
# LN gamma = 1 + N(0, std^2), beta = N(0, std^2).  "scaled" recipe: matrices ~
# N(0, 1/fan_in) so every sub-block contributes O(1) (used by parity tests so that a
# wrong attention/MLP term cannot hide under the residual stream).
# --------------------------------------------------------------------------------------

def make_weights(m: ModelShape, seed: int = 0, dtype: str = "fp16", recipe: str = "paper",
                 std: float = 0.02) -> "OrderedDict[str, np.ndarray]":
    shapes = hf_param_shapes(m)
    ss = np.random.SeedSequence(seed)
    children = ss.spawn(len(shapes))
    out: "OrderedDict[str, np.ndarray]" = OrderedDict()
    for (name, shape), child in zip(shapes.items(), children):
        rng = np.random.Generator(np.random.PCG64(child))
        is_ln = ("LayerNorm" in name) or (".ln_" in name) or name.startswith("ln_")
        if is_ln and name.endswith("weight"):
            a = 1.0 + std * rng.standard_normal(shape, dtype=np.float32)
        elif recipe == "scaled" and len(shape) == 2 and "embeddings" not in name \
                and not name.startswith(("wte", "wpe")):
            # fan_in: HF Linear [out,in] -> shape[1]; GPT-2 Conv1D [in,out] -> shape[0]
            fan_in = shape[0] if m.family == "gpt2" else shape[1]
            a = rng.standard_normal(shape, dtype=np.float32) / np.sqrt(fan_in)
        elif recipe == "scaled" and len(shape) == 2:
            a = rng.standard_normal(shape, dtype=np.float32)  # embeddings O(1)
        elif recipe == "scaled":
            a = 0.1 * rng.standard_normal(shape, dtype=np.float32)
        else:
            a = std * rng.standard_normal(shape, dtype=np.float32)
        out[name] = round_to(a, dtype)
    return out


def make_ids(m: ModelShape, batch: int, seq: int, seed: int = 1) -> np.ndarray:
    """Token ids: U[0,V) for BERT/GPT-2, U[3,V) for RoBERTa (no pad=1)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    lo = 3 if m.family == "roberta" else 0
    return rng.integers(lo, m.vocab, size=(batch, seq), dtype=np.int64).astype(np.int32)


# --------------------------------------------------------------------------------------
# Planner inputs: random int64 cost tables (ns).  Layout: dict of int64 arrays.
# --------------------------------------------------------------------------------------

INF_NS = 1 << 50  # DP_INF: marks DHA-ineligible units


def make_cost_table(n: int, seed: int, *, max_ns: int = 1000, p_inf: float = 0.0,
                    neg_pd: bool = True) -> dict:
    rng = np.random.Generator(np.random.PCG64(seed))
    bytes_ = rng.integers(1, 1 << 20, size=n, dtype=np.int64)
    load = rng.integers(0, max_ns, size=n, dtype=np.int64)
    fwd = rng.integers(0, max_ns // 4 + 1, size=n, dtype=np.int64)
    exe_mem = rng.integers(0, max_ns, size=n, dtype=np.int64)
    lo = -exe_mem if neg_pd else np.zeros(n, dtype=np.int64)
    exe_dha = exe_mem + rng.integers(0, max_ns, size=n, dtype=np.int64) + \
        np.where(rng.random(n) < 0.2, lo // 2, 0)
    exe_dha = np.maximum(exe_dha, 0)
    if p_inf > 0:
        exe_dha = np.where(rng.random(n) < p_inf, INF_NS, exe_dha)
    # link time of a unit's DHA reads: mostly below its load time (embedding-like), sometimes
    # about equal or above it (linear-like: every weight byte crosses the link anyway)
    dha_link = (load * rng.integers(0, 130, size=n) // 100).astype(np.int64)
    return {"bytes": bytes_, "load_ns": load, "fwd_ns": fwd, "exe_mem_ns": exe_mem,
            "exe_dha_ns": exe_dha.astype(np.int64), "dha_link_ns": dha_link}


# --------------------------------------------------------------------------------------
# Serving traces (Poisson arrivals, instance chosen uniformly at random)
# --------------------------------------------------------------------------------------

def make_poisson_trace(n_req: int, rate_per_s: float, n_instances: int, seed: int = 7,
                       mix: "list[float] | None" = None, model_of_instance: "np.ndarray | None" = None):
    """Returns (arrival_ns int64[n], instance int32[n]).

    Inter-arrival times ~ Exp(rate); each request picks an instance uniformly.
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    gaps = rng.exponential(1.0 / rate_per_s, size=n_req)
    t = np.cumsum(gaps)
    arrival_ns = np.round(t * 1e9).astype(np.int64)
    inst = rng.integers(0, n_instances, size=n_req, dtype=np.int64).astype(np.int32)
    return arrival_ns, inst


def make_maf_like_trace(duration_s: float, rate_per_s: float, n_instances: int, seed: int = 7, *,
                        zipf_a: float = 1.1, swing: float = 0.5, period_s: float | None = None,
                        spikes_per_min: float = 6.0, spike_s: float = 1.5, spike_gain: float = 20.0,
                        spike_frac: float = 0.05, bin_s: float = 0.05):
    """A synthetic stand-in for the Azure Functions (MAF) trace of P:342-350 (the real trace
    is not available offline): "heavy sustained requests, fluctuations in request rates, and
    spikes in requests", mapped to the n instances.

    * popularity: instance i gets share ~ 1 / (rank_i)^zipf_a (a random permutation of ranks),
      so a few instances are hot and sustained and most are rare;
    * fluctuation: the offered load is rate * (1 + swing * sin(2 pi t / period)) (period =
      duration / 3 by default);
    * spikes: Poisson spike events (spikes_per_min); each multiplies the rate of a random
      spike_frac of the instances by spike_gain for spike_s seconds.
    The base load is normalised so the mean offered rate (without spikes) is rate_per_s.
    Arrivals are a piecewise-constant-rate Poisson process on bins of bin_s seconds.
    Returns (arrival_ns int64[n], instance int32[n]), sorted by arrival."""
    rng = np.random.Generator(np.random.PCG64(seed))
    period_s = period_s or duration_s / 3.0
    ranks = rng.permutation(n_instances) + 1
    share = 1.0 / ranks.astype(np.float64) ** zipf_a
    share /= share.sum()
    nb = int(np.ceil(duration_s / bin_s))
    t0 = np.arange(nb) * bin_s
    g = 1.0 + swing * np.sin(2 * np.pi * (t0 + 0.5 * bin_s) / period_s)
    lam = np.outer(g * rate_per_s * bin_s, share)  # [bins, instances] expected counts
    n_spikes = rng.poisson(spikes_per_min * duration_s / 60.0)
    for _ in range(n_spikes):
        start = rng.uniform(0, duration_s)
        b0, b1 = int(start / bin_s), int(min(duration_s, start + spike_s) / bin_s) + 1
        hot = rng.choice(n_instances, size=max(1, int(round(spike_frac * n_instances))), replace=False)
        lam[b0:b1, hot] *= spike_gain
    counts = rng.poisson(lam)
    times, insts = [], []
    for b in range(nb):
        row = counts[b]
        nz = np.nonzero(row)[0]
        for i in nz:
            k = int(row[i])
            times.append(t0[b] + rng.uniform(0, bin_s, size=k))
            insts.append(np.full(k, i, dtype=np.int32))
    if not times:
        return np.zeros(0, np.int64), np.zeros(0, np.int32)
    t = np.concatenate(times)
    inst = np.concatenate(insts)
    order = np.argsort(t, kind="stable")
    return np.round(t[order] * 1e9).astype(np.int64), inst[order]


def instance_models(n_instances: int, ratio=(4, 4, 1)) -> np.ndarray:
    """Model index per instance following a mix ratio (4:4:1 BERT/RoBERTa/GPT-2)."""
    tot = sum(ratio)
    out = np.empty(n_instances, dtype=np.int32)
    for i in range(n_instances):
        r = i % tot
        acc = 0
        for k, w in enumerate(ratio):
            acc += w
            if r < acc:
                out[i] = k
                break
    return out
