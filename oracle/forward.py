"""ORACLE (test infrastructure): fp64 reference forward of the paper's transformer models.

PAPER.md P:241 evaluates BERT-Base/Large, RoBERTa-Base/Large, GPT-2/GPT-2 Medium "from
Transformers [35]"; DeepPlan changes only where each layer's weights are read from
(host memory via direct-host-access, or GPU memory after loading), never
the arithmetic.  So this is the plain HF definition, written out step by step
(SURVEY §8(c) "F. Forward"):

BERT / RoBERTa
  e = word[ids] + pos[p] + type[0]      p = arange(S) (BERT) | pad_idx+1+arange(S) (RoBERTa)
  x = LN(e)
  per layer: q,k,v = x Wq^T + bq, ...; a = softmax(q k^T / sqrt(d)); c = a v
             x1 = LN(x + c Wo^T + bo);  h = gelu_erf(x1 W1^T + b1);  x = LN(x1 + h W2^T + b2)
  pooled = tanh(x[:,0] Wp^T + bp)
GPT-2 (pre-LN, Conv1D weights are [in, out])
  x = wte[ids] + wpe[arange(S)]
  per block: x += c_proj(attn_causal(c_attn(LN1(x)))); x += proj2(gelu_tanh(fc(LN2(x))))
  x = ln_f(x)

All arithmetic is float64 on the storage-rounded weights (fp16/bf16/fp32 -> f64).  The one
exception is `forward(..., compute="f32")`: the same definition evaluated in numpy float32, the
"numpy fp32 forward" SURVEY §8(d) times as the CPU baseline beside the GPU (never a parity
reference).  And `forward(..., act_round="bf16")`: the same definition with the activations
rounded to a 16-bit type exactly where a pipeline that stores them in that type must round them
(every linear's input operand, the attention inputs q / k / v, the softmax numerators before P.V,
the output) and nothing else (residual sums stay exact).  It measures the REPRESENTATION error
of storing activations in that type -- the bf16 tolerance is set from it (R15).
"""
from __future__ import annotations

import math

import numpy as np
from scipy.special import erf

from synth import ModelShape, round_to, storage_to_f64


def layer_norm(x: np.ndarray, gamma: np.ndarray, beta: np.ndarray, eps: float) -> np.ndarray:
    """LN over the last axis ("layer normalization"), biased variance, HF eps."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * gamma + beta


def gelu_erf(x: np.ndarray) -> np.ndarray:
    """BERT/RoBERTa GELU: 0.5 x (1 + erf(x / sqrt 2))."""
    return 0.5 * x * (1.0 + erf(x / math.sqrt(2.0)))


def gelu_tanh(x: np.ndarray) -> np.ndarray:
    """GPT-2 GELU ("gelu_new"): 0.5 x (1 + tanh(sqrt(2/pi) (x + 0.044715 x^3)))."""
    return 0.5 * x * (1.0 + np.tanh(math.sqrt(2.0 / math.pi) * (x + 0.044715 * x ** 3)))


def softmax(z: np.ndarray) -> np.ndarray:
    z = z - z.max(axis=-1, keepdims=True)
    e = np.exp(z)
    return e / e.sum(axis=-1, keepdims=True)


def _rnd(x: np.ndarray, dtype) -> np.ndarray:
    """Round to a 16-bit storage type (RNE) and back; identity when dtype is None."""
    if dtype is None:
        return x
    return storage_to_f64(round_to(np.asarray(x, dtype=np.float32), dtype), dtype).astype(x.dtype, copy=False)


def attention(q: np.ndarray, k: np.ndarray, v: np.ndarray, heads: int, causal: bool, p_round=None) -> np.ndarray:
    """Multi-head scaled dot-product attention. q,k,v: [B,S,H] -> [B,S,H].  p_round: the storage
    type the softmax numerators exp(s - max) are rounded to before P.V (the row sums are not)."""
    B, S, H = q.shape
    d = H // heads
    qh = q.reshape(B, S, heads, d).transpose(0, 2, 1, 3)
    kh = k.reshape(B, S, heads, d).transpose(0, 2, 1, 3)
    vh = v.reshape(B, S, heads, d).transpose(0, 2, 1, 3)
    scores = qh @ kh.transpose(0, 1, 3, 2) / math.sqrt(d)
    if causal:
        mask = np.triu(np.ones((S, S), dtype=bool), k=1)
        scores = np.where(mask, -np.inf, scores)
    if p_round is None:
        p = softmax(scores)
        ctx = p @ vh
    else:
        e = np.exp(scores - scores.max(axis=-1, keepdims=True))
        ctx = (_rnd(e, p_round) @ vh) / e.sum(axis=-1, keepdims=True)
    return ctx.transpose(0, 2, 1, 3).reshape(B, S, H)


def _w(weights, name, dtype):
    return storage_to_f64(weights[name], dtype)


def forward(m: ModelShape, weights, ids: np.ndarray, dtype: str = "fp16", compute: str = "f64",
            act_round: str | None = None):
    """Returns (last_hidden_state [B,S,H], pooled [B,H] or None) in float64 (compute="f64", the
    oracle) or float32 (compute="f32", the CPU-baseline timing variant).  act_round: see the
    module docstring (None = exact)."""
    R = lambda t: _rnd(t, act_round)  # noqa: E731
    ids = np.asarray(ids)
    B, S = ids.shape
    cdt = {"f64": np.float64, "f32": np.float32}[compute]
    cache = {}

    def W(n):
        if n not in cache:
            cache[n] = _w(weights, n, dtype).astype(cdt, copy=False)
        return cache[n]
    if m.family in ("bert", "roberta"):
        if m.family == "bert":
            pos = np.arange(S)
        else:
            pos = m.pad_idx + 1 + np.arange(S)  # RoBERTa position ids (no pad tokens)
        e = W("embeddings.word_embeddings.weight")[ids] \
            + W("embeddings.position_embeddings.weight")[pos][None] \
            + W("embeddings.token_type_embeddings.weight")[0][None, None]
        x = layer_norm(e, W("embeddings.LayerNorm.weight"), W("embeddings.LayerNorm.bias"), m.ln_eps)
        for i in range(m.layers):
            p = f"encoder.layer.{i}."
            lin = lambda t, n: R(t) @ W(p + n + ".weight").T + W(p + n + ".bias")  # noqa: E731
            q = R(lin(x, "attention.self.query"))
            k = R(lin(x, "attention.self.key"))
            v = R(lin(x, "attention.self.value"))
            c = attention(q, k, v, m.heads, causal=False, p_round=act_round)
            x1 = layer_norm(x + lin(c, "attention.output.dense"),
                            W(p + "attention.output.LayerNorm.weight"),
                            W(p + "attention.output.LayerNorm.bias"), m.ln_eps)
            h = gelu_erf(lin(x1, "intermediate.dense"))
            x = layer_norm(x1 + lin(h, "output.dense"), W(p + "output.LayerNorm.weight"),
                           W(p + "output.LayerNorm.bias"), m.ln_eps)
        x = R(x)  # the output itself is stored in the type
        pooled = R(np.tanh(x[:, 0] @ W("pooler.dense.weight").T + W("pooler.dense.bias")))
        return x, pooled
    if m.family == "gpt2":
        x = W("wte.weight")[ids] + W("wpe.weight")[np.arange(S)][None]
        H = m.hidden
        for i in range(m.layers):
            p = f"h.{i}."
            conv = lambda t, n: R(t) @ W(p + n + ".weight") + W(p + n + ".bias")  # noqa: E731
            a = layer_norm(x, W(p + "ln_1.weight"), W(p + "ln_1.bias"), m.ln_eps)
            qkv = R(conv(a, "attn.c_attn"))
            c = attention(qkv[..., :H], qkv[..., H:2 * H], qkv[..., 2 * H:], m.heads, causal=True,
                          p_round=act_round)
            x = x + conv(c, "attn.c_proj")
            a = layer_norm(x, W(p + "ln_2.weight"), W(p + "ln_2.bias"), m.ln_eps)
            x = x + conv(gelu_tanh(conv(a, "mlp.c_fc")), "mlp.c_proj")
        x = R(layer_norm(x, W("ln_f.weight"), W("ln_f.bias"), m.ln_eps))
        return x, None
    raise ValueError(m.family)


def embed(m: ModelShape, weights, ids: np.ndarray, dtype: str = "fp16") -> np.ndarray:
    """The embedding step alone: LN(word+pos+type) or wte+wpe."""
    ids = np.asarray(ids)
    B, S = ids.shape
    W = lambda n: _w(weights, n, dtype)  # noqa: E731
    if m.family == "gpt2":
        return W("wte.weight")[ids] + W("wpe.weight")[np.arange(S)][None]
    pos = np.arange(S) if m.family == "bert" else m.pad_idx + 1 + np.arange(S)
    e = W("embeddings.word_embeddings.weight")[ids] \
        + W("embeddings.position_embeddings.weight")[pos][None] \
        + W("embeddings.token_type_embeddings.weight")[0][None, None]
    return layer_norm(e, W("embeddings.LayerNorm.weight"), W("embeddings.LayerNorm.bias"), m.ln_eps)


def linear(x: np.ndarray, w_nk: np.ndarray, b: np.ndarray | None = None, act: str = "none",
           residual: np.ndarray | None = None) -> np.ndarray:
    """Y = act(X W^T + b) (+ residual) in f64 -- the single-linear oracle for the skinny
    DHA linear and the resident GEMM (a12)."""
    y = x @ w_nk.T
    if b is not None:
        y = y + b
    if act == "gelu_erf":
        y = gelu_erf(y)
    elif act == "gelu_tanh":
        y = gelu_tanh(y)
    elif act == "tanh":
        y = np.tanh(y)
    if residual is not None:
        y = y + residual
    return y


def lm_head(m: ModelShape, weights, hidden: np.ndarray, dtype: str = "fp16") -> np.ndarray:
    """GPT-2's tied language-model head (the "logits" of P:241 read literally):
    logits = hidden . wte^T over the whole vocabulary, f64.  hidden: [..., H]."""
    if m.family != "gpt2":
        raise ValueError("tied LM head: GPT-2 only")
    return np.asarray(hidden, dtype=np.float64) @ _w(weights, "wte.weight", dtype).T
