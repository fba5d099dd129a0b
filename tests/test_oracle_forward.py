"""Pins for the fp64 forward oracle (oracle/forward.py) against things other than itself:

* transformers 5.5 CPU BertModel / RobertaModel / GPT2Model in float64 with the same
  state dict -- a library routine sharing no code with the oracle;
* brute-force per-element loops for attention and LayerNorm on tiny shapes;
* invariants: softmax rows sum to 1, LN output has mean 0 / var 1 before the affine step;
* Table 1 byte closed forms (tests/golden/table1_pcie_lines.json).
"""
import json
import math
import os

import numpy as np
import pytest

import synth
from oracle import forward as F
from oracle import units as U

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _hf_model(m, weights, dtype):
    import torch
    from transformers import (BertConfig, BertModel, GPT2Config, GPT2Model, RobertaConfig,
                              RobertaModel)
    if m.family == "bert":
        cfg = BertConfig(vocab_size=m.vocab, hidden_size=m.hidden, num_hidden_layers=m.layers,
                         num_attention_heads=m.heads, intermediate_size=m.ffn,
                         max_position_embeddings=m.max_pos, type_vocab_size=m.type_vocab,
                         layer_norm_eps=m.ln_eps, hidden_act="gelu", attn_implementation="eager")
        model = BertModel(cfg)
    elif m.family == "roberta":
        cfg = RobertaConfig(vocab_size=m.vocab, hidden_size=m.hidden, num_hidden_layers=m.layers,
                            num_attention_heads=m.heads, intermediate_size=m.ffn,
                            max_position_embeddings=m.max_pos, type_vocab_size=m.type_vocab,
                            layer_norm_eps=m.ln_eps, hidden_act="gelu", pad_token_id=m.pad_idx,
                            attn_implementation="eager")
        model = RobertaModel(cfg)
    else:
        cfg = GPT2Config(vocab_size=m.vocab, n_embd=m.hidden, n_layer=m.layers, n_head=m.heads,
                         n_positions=m.max_pos, n_inner=m.ffn, activation_function="gelu_new",
                         layer_norm_epsilon=m.ln_eps, resid_pdrop=0.0, embd_pdrop=0.0,
                         attn_pdrop=0.0, attn_implementation="eager")
        model = GPT2Model(cfg)
    model = model.double().eval()
    sd = {k: torch.from_numpy(synth.storage_to_f64(v, dtype)) for k, v in weights.items()}
    missing, unexpected = model.load_state_dict(sd, strict=False)
    assert not unexpected, unexpected
    # only non-parameter buffers may be missing
    params = dict(model.named_parameters())
    assert not [k for k in missing if k in params], missing
    return model


@pytest.mark.parametrize("name", ["tiny_bert", "tiny_roberta", "tiny_gpt2"])
@pytest.mark.parametrize("recipe", ["paper", "scaled"])
def test_forward_matches_transformers(name, recipe):
    import torch
    m = synth.SHAPES[name]
    dtype = "fp16"
    w = synth.make_weights(m, seed=3, dtype=dtype, recipe=recipe)
    ids = synth.make_ids(m, 2, 37, seed=5)
    x, pooled = F.forward(m, w, ids, dtype)
    model = _hf_model(m, w, dtype)
    with torch.no_grad():
        kw = {}
        if m.family != "gpt2":
            kw["token_type_ids"] = torch.zeros(ids.shape, dtype=torch.long)
            kw["attention_mask"] = torch.ones(ids.shape, dtype=torch.long)
        out = model(input_ids=torch.from_numpy(ids.astype(np.int64)), **kw)
    ref = out.last_hidden_state.numpy()
    assert np.max(np.abs(x - ref)) < 1e-9
    if m.family != "gpt2":
        assert np.max(np.abs(pooled - out.pooler_output.numpy())) < 1e-9


def test_forward_bert_base_matches_transformers_short():
    """A full-size BERT-Base (12 layers, H=768) on a short sequence."""
    import torch
    m = synth.SHAPES["bert_base"]
    w = synth.make_weights(m, seed=11, dtype="fp16")
    ids = synth.make_ids(m, 1, 16, seed=2)
    x, pooled = F.forward(m, w, ids, "fp16")
    model = _hf_model(m, w, "fp16")
    with torch.no_grad():
        out = model(input_ids=torch.from_numpy(ids.astype(np.int64)),
                    token_type_ids=torch.zeros(ids.shape, dtype=torch.long))
    assert np.max(np.abs(x - out.last_hidden_state.numpy())) < 1e-9
    assert np.max(np.abs(pooled - out.pooler_output.numpy())) < 1e-9


def test_bf16_weights_decode():
    m = synth.SHAPES["tiny_bert"]
    w16 = synth.make_weights(m, seed=3, dtype="bf16")
    w32 = synth.make_weights(m, seed=3, dtype="fp32")
    a = synth.storage_to_f64(w16["embeddings.word_embeddings.weight"], "bf16")
    b = w32["embeddings.word_embeddings.weight"].astype(np.float64)
    # bf16 has 8 mantissa bits: relative rounding error <= 2^-9
    assert np.all(np.abs(a - b) <= np.abs(b) * 2.0 ** -8 + 1e-30)


def test_attention_bruteforce_loops():
    rng = np.random.default_rng(0)
    B, S, H, heads = 1, 5, 8, 2
    q, k, v = (rng.standard_normal((B, S, H)) for _ in range(3))
    for causal in (False, True):
        got = F.attention(q, k, v, heads, causal)
        d = H // heads
        ref = np.zeros((B, S, H))
        for h in range(heads):
            for i in range(S):
                sc = []
                for j in range(S):
                    if causal and j > i:
                        continue
                    sc.append(sum(q[0, i, h * d + t] * k[0, j, h * d + t] for t in range(d)) / math.sqrt(d))
                mx = max(sc)
                ex = [math.exp(s - mx) for s in sc]
                z = sum(ex)
                for t in range(d):
                    ref[0, i, h * d + t] = sum(ex[j] / z * v[0, j, h * d + t] for j in range(len(ex)))
        assert np.max(np.abs(got - ref)) < 1e-12


def test_softmax_rows_sum_to_one():
    rng = np.random.default_rng(1)
    p = F.softmax(rng.standard_normal((7, 33)) * 10)
    assert np.allclose(p.sum(-1), 1.0, atol=1e-12)
    assert np.all(p >= 0)


def test_layernorm_bruteforce_and_invariants():
    rng = np.random.default_rng(2)
    x = rng.standard_normal((3, 11)) * 4 + 2
    g, b = np.ones(11), np.zeros(11)
    y = F.layer_norm(x, g, b, 1e-12)
    assert np.allclose(y.mean(-1), 0, atol=1e-12)
    assert np.allclose(y.var(-1), 1, atol=1e-9)
    g2, b2 = rng.standard_normal(11), rng.standard_normal(11)
    y2 = F.layer_norm(x, g2, b2, 1e-5)
    for r in range(3):
        mu = sum(x[r]) / 11
        var = sum((t - mu) ** 2 for t in x[r]) / 11
        for c in range(11):
            assert abs(y2[r, c] - ((x[r, c] - mu) / math.sqrt(var + 1e-5) * g2[c] + b2[c])) < 1e-12


def test_gelu_special_values():
    assert F.gelu_erf(np.array([0.0]))[0] == 0.0
    # gelu(x) - gelu(-x) = x  (odd part), both variants
    x = np.linspace(-5, 5, 41)
    assert np.allclose(F.gelu_erf(x) - F.gelu_erf(-x), x, atol=1e-12)
    assert np.allclose(F.gelu_tanh(x) - F.gelu_tanh(-x), x, atol=1e-12)
    # large x: gelu(x) ~ x
    assert abs(F.gelu_erf(np.array([10.0]))[0] - 10.0) < 1e-12


def test_embed_matches_forward_prefix():
    m = synth.SHAPES["tiny_bert"]
    w = synth.make_weights(m, seed=4)
    ids = synth.make_ids(m, 1, 9)
    e = F.embed(m, w, ids)
    # an L=0 model's output equals the embedding step
    import dataclasses
    m0 = dataclasses.replace(m, layers=0)
    w0 = {k: v for k, v in w.items() if not k.startswith("encoder.")}
    x, _ = F.forward(m0, w0, ids)
    assert np.array_equal(e, x)


def test_table1_closed_forms():
    """Table 1: load lines = bytes/64 and DHA embedding lines = S*H*4/64
    reproduce the paper's measured counts to within 0.25% (BERT-Base, fp32, S=384)."""
    gold = json.load(open(os.path.join(GOLD, "table1_pcie_lines.json")))
    m = synth.SHAPES["bert_base"]
    ub = dict(zip([u[0] for u in U.unit_params(m)], U.unit_bytes(m, "fp32")))
    S = gold["seq_len"]
    pred_load = [U.pcie_lines_load(ub["pos"]), U.pcie_lines_load(ub["word"]),
                 U.pcie_lines_load(ub["L0.q"]), U.pcie_lines_load(ub["L0.fc1"])]
    for row, p in zip(gold["rows"], pred_load):
        assert abs(p - row["load"]) / row["load"] < 2.5e-3, (row, p)
    # DHA word embedding: S rows touched
    dha_word = U.pcie_lines_dha_gather(S, m.hidden, "fp32")
    assert abs(dha_word - gold["rows"][1]["dha"]) / gold["rows"][1]["dha"] < 2.5e-3
    # DHA on FC reads far more than the layer (reuse across tokens): > 10x the load lines
    assert gold["rows"][2]["dha"] > 10 * pred_load[2]
    # 89.4MB word embedding out of 417MB (MiB) for fp32 BERT-Base
    assert round(U.model_bytes(m, "fp32") / 2 ** 20) == gold["model_total_MB"] + 1 or \
        int(U.model_bytes(m, "fp32") / 2 ** 20) == gold["model_total_MB"]
    assert abs(ub["word"] / 2 ** 20 - gold["word_embedding_MB"]) < 0.05


def test_unit_counts_and_fp16_bytes():
    """unit counts and fp16 model bytes."""
    expect = {"tiny_bert": (21, 1_214_208), "bert_base": (101, 218_964_480),
              "bert_large": (197, 670_283_776), "roberta_large": (197, 710_719_488),
              "gpt2_medium": (147, 709_646_336)}
    for name, (n, nb) in expect.items():
        m = synth.SHAPES[name]
        assert len(U.unit_params(m)) == n
        assert U.model_bytes(m, "fp16") == nb


def test_lm_head_matches_transformers_gpt2_lm_head():
    """The oracle's tied LM head = transformers' GPT2LMHeadModel logits (same state dict, f64)."""
    import torch
    from transformers import GPT2Config, GPT2LMHeadModel
    m = synth.SHAPES["tiny_gpt2"]
    dtype = "fp16"
    w = synth.make_weights(m, seed=9, dtype=dtype)
    ids = synth.make_ids(m, 2, 19, seed=4)
    x, _ = F.forward(m, w, ids, dtype)
    logits = F.lm_head(m, w, x, dtype)
    cfg = GPT2Config(vocab_size=m.vocab, n_embd=m.hidden, n_layer=m.layers, n_head=m.heads, n_positions=m.max_pos,
                     n_inner=m.ffn, activation_function="gelu_new", layer_norm_epsilon=m.ln_eps, resid_pdrop=0.0,
                     embd_pdrop=0.0, attn_pdrop=0.0, attn_implementation="eager", tie_word_embeddings=True)
    model = GPT2LMHeadModel(cfg).double().eval()
    sd = {"transformer." + k: torch.from_numpy(synth.storage_to_f64(v, dtype)) for k, v in w.items()}
    missing, unexpected = model.load_state_dict(sd, strict=False)
    assert not unexpected, unexpected
    assert model.lm_head.weight.data_ptr() == model.transformer.wte.weight.data_ptr()  # tied
    with torch.no_grad():
        ref = model(input_ids=torch.from_numpy(ids.astype(np.int64))).logits.numpy()
    assert logits.shape == (2, 19, m.vocab)
    assert np.max(np.abs(logits - ref)) < 1e-9
    with pytest.raises(ValueError):
        F.lm_head(synth.SHAPES["tiny_bert"], w, x, dtype)
