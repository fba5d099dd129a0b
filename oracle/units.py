"""ORACLE (test infrastructure): planning units and byte accounting.

A planning unit is one weight-bearing leaf module (Table 3 P:257-263 lists
"Emb", "LN", "FC" as the paper's layers).  Parameterless ops (attention core, GELU,
residual) are charged to the preceding unit.

BERT/RoBERTa: word, pos, type, emb_ln, per layer {q,k,v,attn_out,ln1,fc1,fc2,ln2}, pooler
GPT-2:        wte, wpe, per block {ln_1,c_attn,c_proj,ln_2,c_fc,mlp_c_proj}, ln_f

Bytes of a unit = sum of its parameters' storage bytes (weight then bias / gamma then
beta).  Table 1 pins this: "the number of PCIe accesses is that the layer
size is divided by 64B" for a load, and a DHA gather touches only the used rows.
"""
from __future__ import annotations

from synth import ModelShape, hf_param_shapes

DTYPE_BYTES = {"fp16": 2, "bf16": 2, "fp32": 4}


def unit_params(m: ModelShape):
    """[(unit_name, kind, [hf param names])] in forward order."""
    u = []
    if m.family in ("bert", "roberta"):
        u.append(("word", "emb", ["embeddings.word_embeddings.weight"]))
        u.append(("pos", "emb", ["embeddings.position_embeddings.weight"]))
        u.append(("type", "emb", ["embeddings.token_type_embeddings.weight"]))
        u.append(("emb_ln", "ln", ["embeddings.LayerNorm.weight", "embeddings.LayerNorm.bias"]))
        for i in range(m.layers):
            p = f"encoder.layer.{i}."
            for short, mod in (("q", "attention.self.query"), ("k", "attention.self.key"),
                               ("v", "attention.self.value"), ("attn_out", "attention.output.dense")):
                u.append((f"L{i}.{short}", "linear", [p + mod + ".weight", p + mod + ".bias"]))
            u.append((f"L{i}.ln1", "ln", [p + "attention.output.LayerNorm.weight",
                                           p + "attention.output.LayerNorm.bias"]))
            u.append((f"L{i}.fc1", "linear", [p + "intermediate.dense.weight", p + "intermediate.dense.bias"]))
            u.append((f"L{i}.fc2", "linear", [p + "output.dense.weight", p + "output.dense.bias"]))
            u.append((f"L{i}.ln2", "ln", [p + "output.LayerNorm.weight", p + "output.LayerNorm.bias"]))
        u.append(("pooler", "linear", ["pooler.dense.weight", "pooler.dense.bias"]))
    else:
        u.append(("wte", "emb", ["wte.weight"]))
        u.append(("wpe", "emb", ["wpe.weight"]))
        for i in range(m.layers):
            p = f"h.{i}."
            u.append((f"L{i}.ln_1", "ln", [p + "ln_1.weight", p + "ln_1.bias"]))
            u.append((f"L{i}.c_attn", "linear", [p + "attn.c_attn.weight", p + "attn.c_attn.bias"]))
            u.append((f"L{i}.c_proj", "linear", [p + "attn.c_proj.weight", p + "attn.c_proj.bias"]))
            u.append((f"L{i}.ln_2", "ln", [p + "ln_2.weight", p + "ln_2.bias"]))
            u.append((f"L{i}.c_fc", "linear", [p + "mlp.c_fc.weight", p + "mlp.c_fc.bias"]))
            u.append((f"L{i}.mlp_c_proj", "linear", [p + "mlp.c_proj.weight", p + "mlp.c_proj.bias"]))
        u.append(("ln_f", "ln", ["ln_f.weight", "ln_f.bias"]))
    return u


def unit_bytes(m: ModelShape, dtype: str = "fp16") -> list[int]:
    shapes = hf_param_shapes(m)
    eb = DTYPE_BYTES[dtype]
    out = []
    for _, _, params in unit_params(m):
        n = 0
        for p in params:
            c = 1
            for d in shapes[p]:
                c *= d
            n += c * eb
        out.append(n)
    return out


def model_bytes(m: ModelShape, dtype: str = "fp16") -> int:
    return sum(unit_bytes(m, dtype))


def pcie_lines_load(nbytes: int, line: int = 64) -> int:
    """Table 1: a load moves the layer in 64 B PCIe payloads -> bytes/64."""
    return -(-nbytes // line)


def pcie_lines_dha_gather(rows_touched: int, hidden: int, dtype: str = "fp32", line: int = 64) -> int:
    """Table 1: a DHA embedding touches only the used rows: rows * row bytes / 64."""
    return -(-rows_touched * hidden * DTYPE_BYTES[dtype] // line)
