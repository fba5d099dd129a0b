"""Output precision of full-size cold starts per storage dtype ("measure and print
bf16 max-abs with the fp32 residual stream"), R15.

For each paper model at its config's sequence length: one cold start with every unit loaded (all
linears on the tcgen05 GEMM) compared element by element with
  * the exact oracle (fp64 on the storage-rounded weights), and
  * the oracle with the activations rounded to the storage type exactly where the kernels must
    store them in it (every linear's input, q / k / v, the softmax numerators, the output;
    oracle.forward act_round) -- the error a 16-bit activation type causes by itself.
fp16 meets the north star's max-abs 1e-2 against the exact oracle outright.  bf16 cannot: its
representation error alone is 0.017-0.022 on these models (8 fewer significand bits than fp16's
10 + 1; the fp16 representation error is 0.002-0.003), so for bf16 the north star's 1e-2 is
applied to what the kernels add -- |gpu - emulated| <= 1e-2 -- and against the exact oracle the
bound is 1e-2 + the representation error.  Set DP_PRECISION_OUT=file.jsonl to record the values.
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
    if dtype == "fp16":
        assert row["max_abs_vs_exact"] <= 1e-2
        assert row.get("pooler_vs_exact", 0) <= 1e-2
    else:
        assert row["max_abs_vs_emulated"] <= 1e-2
        assert row["max_abs_vs_exact"] <= 1e-2 + row["representation_error"]
        assert row.get("pooler_vs_emulated", 0) <= 1e-2
