"""Output precision of full-size cold starts per storage dtype ("measure and print
bf16 max-abs with the fp32 residual stream"), R15.

For each paper model at its config's sequence length: one cold start with every unit loaded (all
linears on the tcgen05 GEMM) compared element by element with
  * the exact oracle (fp64 on the storage-rounded weights), and
  * the oracle with the activations rounded to the storage type exactly where the kernels must
    store them in it (every linear's input, q / k / v, the softmax numerators, the output;
    oracle.forward act_round) -- the error a 16-bit activation type causes by itself.
fp16 meets the north star's max-abs 1e-2 against the exact oracle outright.  bf16 cannot: its
representation error alone is 0.017-0.025 on these models (3 fewer significand bits than fp16;
the fp16 representation error is 0.002-0.003).  Measured on B200 the GPU's error against the
exact oracle is at most the representation error in both dtypes (e.g. BERT-Large bf16 0.0192 vs
0.0218): the kernels add nothing beyond what storing activations in the type costs.  The GPU and
the emulated pipeline round independently, so they differ from each other by about as much again
(reported, not bounded).  Bounds: fp16 max-abs <= 1e-2; both dtypes <= 1.25 x the representation
error + 1e-3; bf16 <= 1e-2 + the representation error (R15).  Set
DP_PRECISION_OUT=file.jsonl to record the values.
"""
import json
import os

import numpy as np
import pytest

import synth
from oracle import forward as F

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TDT = {"fp16": torch.float16, "bf16": torch.bfloat16}


@pytest.mark.parametrize("name,S", [("bert_base", 128), ("bert_large", 384), ("roberta_large", 384),
                                    ("gpt2_medium", 1024)])
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_full_size_precision(name, S, dtype):
    import paper_conf_eurosys_jeongba23_b200 as dp
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=0, dtype=dtype)
    ids = synth.make_ids(m, 1, S, seed=1)
    exact, exact_pool = F.forward(m, w, ids, dtype)
    emul, emul_pool = F.forward(m, w, ids, dtype, act_round=dtype)
    exact, emul = exact.reshape(S, -1), emul.reshape(S, -1)
    c = dp.Context([0])
    model = dp.Model(c, m, w, dtype)
    n = model.n
    plan = dp._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1)
    out = torch.empty(S, m.hidden, dtype=TDT[dtype], device="cuda")
    pool = torch.empty(1, m.hidden, dtype=TDT[dtype], device="cuda") if m.family != "gpt2" else None
    model.infer_cold(plan, 0, torch.from_numpy(ids).cuda(), out, pool)
    torch.cuda.synchronize()
    model.evict(0)
    model.close()
    c.close()
    got = out.double().cpu().numpy()
    row = {"model": name, "seq": S, "dtype": dtype, "max_abs_vs_exact": float(np.abs(got - exact).max()),
           "max_abs_vs_emulated": float(np.abs(got - emul).max()),
           "representation_error": float(np.abs(emul - exact).max())}
    if pool is not None:
        gp = pool.double().cpu().numpy()
        row["pooler_vs_exact"] = float(np.abs(gp - exact_pool).max())
        row["pooler_vs_emulated"] = float(np.abs(gp - emul_pool).max())
    print(json.dumps(row))
    if os.environ.get("DP_PRECISION_OUT"):
        with open(os.environ["DP_PRECISION_OUT"], "a") as f:
            f.write(json.dumps(row) + "\n")
    assert row["max_abs_vs_exact"] <= 1.25 * row["representation_error"] + 1e-3
    if dtype == "fp16":
        assert row["max_abs_vs_exact"] <= 1e-2
        assert row.get("pooler_vs_exact", 0) <= 1e-2
    else:
        assert row["max_abs_vs_exact"] <= 1e-2 + row["representation_error"]
        assert row.get("pooler_vs_exact", 0) <= 1e-2
