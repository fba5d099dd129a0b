"""K6, the persistent layer-program kernel (every layer of a warm forward in one cooperative
launch), against the fp64 oracle through the C-ABI.

* warm forward with opts.persistent = 1 after a cold start that loaded every unit: outputs
  within the north_star tolerance of the oracle (tiny shapes with several tiles and ragged
  token tails, both weight recipes, fp16 / bf16; BERT-Base and GPT-2 at full size);
* the path really ran: 2 kernels (+ pooler) instead of 7 per layer;
* deterministic: repeated runs and CUDA-graph replay are bit-identical (split-K partials are
  summed in split order, no atomics);
* a plan with DHA layer units falls back to the per-kernel path (K6 needs resident weights).
"""
import numpy as np
import pytest

import synth
from oracle import forward as F

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

DT = {"fp16": torch.float16, "bf16": torch.bfloat16}


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def f64(t):
    return t.float().cpu().numpy().astype(np.float64)


def tolerance(dtype, recipe, ref):
    """Same bounds as test_gpu_forward.tolerance."""
    base = np.full_like(ref, 1e-2) if dtype == "fp16" else 2.0 ** -5 * np.maximum(1.0, np.abs(ref))
    return base if recipe == "paper" else 3 * base


def load_all(model, m, ids_t, dtype, B, S):
    """Cold start with every unit loaded (PIPESWITCH plan): the model becomes resident with
    all layer units in HBM."""
    n = model.n
    plan = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), np.zeros(n, np.int8), 1, 1)
    out = torch.empty(B * S, m.hidden, dtype=DT[dtype], device="cuda")
    pool = torch.empty(B, m.hidden, dtype=DT[dtype], device="cuda") if m.family != "gpt2" else None
    model.infer_cold(plan, 0, ids_t, out, pool)
    torch.cuda.synchronize()
    return out, pool


def warm(model, m, ids_t, dtype, B, S):
    out = torch.empty(B * S, m.hidden, dtype=DT[dtype], device="cuda")
    pool = torch.empty(B, m.hidden, dtype=DT[dtype], device="cuda") if m.family != "gpt2" else None
    st = model.infer_warm(0, ids_t, out, pool)
    torch.cuda.synchronize()
    return out, pool, st


CASES = [("tiny_bert", 1, 32), ("tiny_bert", 2, 77), ("tiny_roberta", 2, 50), ("tiny_gpt2", 2, 70),
         ("tiny_gpt2", 1, 200), ("tiny_bert", 3, 130)]


@pytest.mark.parametrize("name,B,S", CASES)
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("recipe", ["paper", "scaled"])
def test_persistent_warm_matches_oracle(name, B, S, dtype, recipe):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=21, dtype=dtype, recipe=recipe)
    ids = synth.make_ids(m, B, S, seed=22)
    ref, ref_pool = F.forward(m, w, ids, dtype)
    ref = ref.reshape(B * S, m.hidden)
    ctx = dp().Context([0])
    model = dp().Model(ctx, m, w, dtype)
    ids_t = torch.from_numpy(ids).cuda()
    base, base_pool = load_all(model, m, ids_t, dtype, B, S)
    ctx.set_opts(persistent=True)
    out, pool, st = warm(model, m, ids_t, dtype, B, S)
    assert st["n_kernels"] == 2 + (1 if pool is not None else 0), st
    err = np.abs(f64(out) - ref)
    assert np.all(err <= tolerance(dtype, recipe, ref)), err.max()
    if pool is not None:
        assert np.all(np.abs(f64(pool) - ref_pool) <= tolerance(dtype, recipe, ref_pool))
    # same math as the per-kernel path, different summation order: close, not identical
    assert np.abs(f64(out) - f64(base)).max() <= 2 * tolerance(dtype, recipe, ref).max()
    # deterministic
    out2, pool2, _ = warm(model, m, ids_t, dtype, B, S)
    assert torch.equal(out, out2)
    model.close()
    ctx.close()


@pytest.mark.parametrize("name,S", [("bert_base", 128), ("gpt2", 256)])
def test_persistent_full_size(name, S):
    """BERT-Base at the bench configuration (configs[1]: batch 1, seq 128) and GPT-2 small."""
    m = synth.SHAPES[name]
    dtype = "fp16"
    w = synth.make_weights(m, seed=0, dtype=dtype)
    ids = synth.make_ids(m, 1, S, seed=1)
    ref, ref_pool = F.forward(m, w, ids, dtype)
    ctx = dp().Context([0])
    model = dp().Model(ctx, m, w, dtype)
    ids_t = torch.from_numpy(ids).cuda()
    load_all(model, m, ids_t, dtype, 1, S)
    ctx.set_opts(persistent=True)
    out, pool, st = warm(model, m, ids_t, dtype, 1, S)
    assert st["n_kernels"] <= 3
    assert np.abs(f64(out) - ref.reshape(S, -1)).max() <= 1e-2
    if pool is not None:
        assert np.abs(f64(pool) - ref_pool).max() <= 1e-2
    model.close()
    ctx.close()


def test_persistent_graph_replay_bit_identical():
    m = synth.SHAPES["tiny_bert"]
    dtype = "fp16"
    w = synth.make_weights(m, seed=5, dtype=dtype, recipe="scaled")
    ids = synth.make_ids(m, 2, 64, seed=6)
    ctx = dp().Context([0])
    model = dp().Model(ctx, m, w, dtype)
    ids_t = torch.from_numpy(ids).cuda()
    load_all(model, m, ids_t, dtype, 2, 64)
    ctx.set_opts(persistent=True, use_graph=False)
    eager, pe, _ = warm(model, m, ids_t, dtype, 2, 64)
    ctx.set_opts(use_graph=True)
    for _ in range(3):
        g, pg, _ = warm(model, m, ids_t, dtype, 2, 64)
        assert torch.equal(g, eager) and torch.equal(pg, pe)
    model.close()
    ctx.close()


def test_persistent_falls_back_when_layers_are_dha():
    m = synth.SHAPES["tiny_bert"]
    dtype = "fp16"
    w = synth.make_weights(m, seed=7, dtype=dtype)
    ids = synth.make_ids(m, 1, 40, seed=8)
    ref, _ = F.forward(m, w, ids, dtype)
    ctx = dp().Context([0])
    model = dp().Model(ctx, m, w, dtype)
    n = model.n
    method = np.zeros(n, np.int8)
    method[5] = 1  # a layer-0 linear (k) read from host memory
    plan = dp()._lib.PlanArrays(n, method, np.zeros(n, np.int8), 1, 1)
    ids_t = torch.from_numpy(ids).cuda()
    out = torch.empty(40, m.hidden, dtype=torch.float16, device="cuda")
    pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda")
    model.infer_cold(plan, 0, ids_t, out, pool)
    ctx.set_opts(persistent=True)
    o2, _, st = warm(model, m, ids_t, dtype, 1, 40)
    assert st["n_kernels"] > 3  # per-kernel path
    assert np.abs(f64(o2) - ref.reshape(40, -1)).max() <= 1e-2
    model.close()
    ctx.close()
