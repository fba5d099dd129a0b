"""fp32 storage (DP_FP32): the paper's own precision (Table 1 counts fp32 bytes, P:113-122;
SURVEY §8(d) C1 "tiny BERT, fp32 + fp16").  North star: logits within 1e-4 relative of the
oracle for fp32.  "Relative" is read normwise per element: |y - ref| <= 1e-4 * max(1, |ref|)
(a pure elementwise ratio is undefined where the reference crosses zero; R24).

* every engine option on tiny BERT / RoBERTa / GPT-2 (C1 shapes, PT slots in loopback) vs the
  fp64 oracle, plus the per-link bytes of the oracle simulator bit-exactly;
* DHA vs loaded execution is bit-identical for EVERY unit kind in fp32 (the fp32 linear is
  one kernel for host-mapped and HBM weights);
* full-size BERT-Base fp32 (S=128) from a live profile, Algorithm-1 plan;
* the fp32 kernels one by one through the C-ABI hooks (linear incl. activations and an
  aliased residual, LayerNorm, attention causal / not, embedding with DHA tables).
"""
import numpy as np
import pytest

import synth
from oracle import forward as F
from oracle import planner as OP
from oracle import units as OU

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

REL = 1e-4


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def f64(t):
    return t.double().cpu().numpy()


def check(y, ref, rel=REL):
    err = np.abs(np.asarray(y, np.float64) - ref)
    bound = rel * np.maximum(1.0, np.abs(ref))
    assert np.all(err <= bound), f"max err {err.max():.3e} (max rel {(err / np.maximum(1, np.abs(ref))).max():.3e})"
    return float(err.max())


def fake_cost(m, seed=0):
    nb = np.array(OU.unit_bytes(m, "fp32"), dtype=np.int64)
    rng = np.random.default_rng(seed)
    n = len(nb)
    load = nb * 1000 // 55_000 + 4000
    exe = rng.integers(3000, 9000, n)
    kinds = [u[1] for u in OU.unit_params(m)]
    dha = np.where(np.array(kinds) == "emb", exe + 2000, exe + load + rng.integers(-6000, 6000, n))
    return {"bytes": nb, "load_ns": load, "fwd_ns": nb // 700, "exe_mem_ns": exe, "exe_dha_ns": np.maximum(dha, 0)}


def run_cold(model, plan, ids_np, secondaries=()):
    H = model.shape.hidden
    B, S = ids_np.shape
    ids = torch.from_numpy(ids_np).cuda()
    out = torch.empty(B * S, H, dtype=torch.float32, device="cuda")
    pool = torch.empty(B, H, dtype=torch.float32, device="cuda") if model.shape.family != "gpt2" else None
    st = model.infer_cold(plan, 0, ids, out, pool, secondaries=secondaries)
    torch.cuda.synchronize()
    return out, pool, st


@pytest.mark.parametrize("name,B,S", [("tiny_bert", 1, 32), ("tiny_bert", 2, 77), ("tiny_roberta", 2, 50),
                                      ("tiny_gpt2", 2, 70)])
@pytest.mark.parametrize("recipe", ["paper", "scaled"])
def test_c1_all_modes_fp32(name, B, S, recipe):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=3, dtype="fp32", recipe=recipe)
    ids = synth.make_ids(m, B, S, seed=4)
    ref, ref_pool = F.forward(m, w, ids, "fp32")
    ref = ref.reshape(B * S, -1)
    c = dp().Context([0])
    model = dp().Model(c, m, w, "fp32")
    cost = fake_cost(m)
    for mode in ("BASELINE", "PIPESWITCH", "GREEDY", "DHA", "PT", "PT_DHA", "DHA_LINK", "PT_DHA_LINK",
                 "PT_DHA_BAL", "PT_DHA_LINK_BAL", "PT_DHA_STRIPE", "PT_DHA_LINK_STRIPE"):
        k = 3 if mode.startswith("PT") else 1
        plan = dp().plan_generate(cost, mode, k)
        out, pool, st = run_cold(model, plan, ids, secondaries=[0] * (k - 1))
        model.evict(0)
        check(f64(out), ref)
        if pool is not None:
            check(f64(pool), ref_pool)
        om, osl, ser = OP.plan(cost, mode, k)
        assert list(plan.method) == om and list(plan.slot) == osl
        link = OP.simulate(cost, om, osl, k if mode.startswith("PT") else 1, ser)["link_bytes"]
        assert st["h2d_bytes"][:len(link)] == link
    model.close()
    c.close()


@pytest.mark.parametrize("name", ["tiny_bert", "tiny_gpt2"])
def test_fp32_dha_vs_load_bit_identical_every_unit(name):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=8, dtype="fp32", recipe="scaled")
    ids = synth.make_ids(m, 1, 40, seed=9)
    c = dp().Context([0])
    model = dp().Model(c, m, w, "fp32")
    n = model.n
    all_load = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1)
    all_dha = dp()._lib.PlanArrays(n, np.ones(n, np.int8), None, 3, 1)
    a, pa, _ = run_cold(model, all_load, ids)
    a = a.clone()
    model.evict(0)
    b, pb, st = run_cold(model, all_dha, ids)
    model.evict(0)
    assert torch.equal(a, b)
    assert st["h2d_bytes"][0] == 0 and st["n_copies"] == 0
    if pa is not None:
        assert torch.equal(pa, pb)
    model.close()
    c.close()


def test_bert_base_fp32_full_size():
    """BERT-Base in the paper's precision: fp32, batch 1, seq 128, live profile -> Algorithm 1."""
    m = synth.SHAPES["bert_base"]
    w = synth.make_weights(m, seed=0, dtype="fp32")
    ids = synth.make_ids(m, 1, 128, seed=1)
    ref, ref_pool = F.forward(m, w, ids, "fp32")
    c = dp().Context([0])
    model = dp().Model(c, m, w, "fp32")
    assert model.nbytes >= 437_000_000  # fp32 BERT-Base (417 MiB)
    cost = model.profile(0, 1, 128, iters=3)
    plan = dp().plan_generate(cost, "DHA", 1)
    assert list(plan.method) == OP.algorithm1(cost)
    out, pool, _ = run_cold(model, plan, ids)
    model.evict(0)
    check(f64(out), ref.reshape(128, -1))
    check(f64(pool), ref_pool)
    model.close()
    c.close()


@pytest.mark.parametrize("act", ["none", "gelu_erf", "gelu_tanh", "tanh"])
@pytest.mark.parametrize("M,N,K", [(1, 768, 768), (37, 200, 64), (128, 3072, 768), (130, 768, 3072)])
def test_fp32_linear_kernel(act, M, N, K):
    rng = np.random.default_rng(M + N + K)
    x = rng.standard_normal((M, K)).astype(np.float32)
    w = (rng.standard_normal((N, K)) / np.sqrt(K)).astype(np.float32)
    b = rng.standard_normal(N).astype(np.float32)
    r = rng.standard_normal((M, N)).astype(np.float32)
    ref = F.linear(x.astype(np.float64), w.astype(np.float64), b.astype(np.float64), act=act,
                   residual=r.astype(np.float64))
    xt, wt, bt = (torch.from_numpy(a).cuda() for a in (x, w, b))
    y = torch.from_numpy(r).cuda()  # residual aliased with the output (GPT-2's in-place stream)
    dp().linear(xt, K, wt, bt, y, N, y, N, M, N, K, act=act, path=1, dtype="fp32")
    torch.cuda.synchronize()
    check(f64(y), ref, rel=1e-5)
    with pytest.raises(dp().DeepPlanError):  # no fp32 tcgen05 kind
        dp().linear(xt, K, wt, bt, None, 0, y, N, M, N, K, act=act, path=0, dtype="fp32")


@pytest.mark.parametrize("B,S,causal", [(1, 32, False), (2, 77, True), (1, 384, False), (1, 1024, True)])
def test_fp32_attention_kernel(B, S, causal):
    heads, H = 4, 256
    rng = np.random.default_rng(S)
    qkv = rng.standard_normal((B * S, 3 * H)).astype(np.float32)
    q, k, v = (qkv[:, i * H:(i + 1) * H].reshape(B, S, H).astype(np.float64) for i in range(3))
    ref = F.attention(q, k, v, heads, causal).reshape(B * S, H)
    out = torch.empty(B * S, H, device="cuda")
    dp().attention(torch.from_numpy(qkv).cuda(), 3 * H, out, B, S, H, heads, causal, dtype="fp32")
    torch.cuda.synchronize()
    check(f64(out), ref, rel=1e-5)


def test_fp32_layernorm_and_embedding_dha():
    m = synth.SHAPES["bert_base"]
    rng = np.random.default_rng(1)
    rows, n = 200, 768
    x = rng.standard_normal((rows, n)).astype(np.float32)
    r = rng.standard_normal((rows, n)).astype(np.float32)
    g = (1 + 0.1 * rng.standard_normal(n)).astype(np.float32)
    b = (0.1 * rng.standard_normal(n)).astype(np.float32)
    ref = F.layer_norm((x + r).astype(np.float64), g.astype(np.float64), b.astype(np.float64), 1e-12)
    y = torch.empty(rows, n, device="cuda")
    gt, bt = torch.from_numpy(g).cuda(), torch.from_numpy(b).cuda()
    dp().layernorm(torch.from_numpy(x).cuda(), torch.from_numpy(r).cuda(), gt, bt, y, rows, n, 1e-12, dtype="fp32")
    torch.cuda.synchronize()
    check(f64(y), ref, rel=1e-5)
    # embedding + LN with every table host-mapped (direct-host-access)
    w = synth.make_weights(m, seed=2, dtype="fp32")
    ids = synth.make_ids(m, 1, 128, seed=3)
    ref_e = F.embed(m, w, ids, "fp32").reshape(128, -1)
    names = ["embeddings.word_embeddings.weight", "embeddings.position_embeddings.weight",
             "embeddings.token_type_embeddings.weight", "embeddings.LayerNorm.weight", "embeddings.LayerNorm.bias"]
    bufs = []
    for nm in names:
        a = np.ascontiguousarray(w[nm])
        p = dp().host_alloc(a.nbytes)
        np.ctypeslib.as_array((np.ctypeslib.ctypes.c_uint8 * a.nbytes).from_address(p))[:] = \
            np.frombuffer(a.tobytes(), dtype=np.uint8)
        bufs.append(p)
    out = torch.empty(128, 768, device="cuda")
    dp().embed(torch.from_numpy(ids).cuda(), 128, *bufs, 768, 1e-12, out, dtype="fp32")
    torch.cuda.synchronize()
    check(f64(out), ref_e, rel=1e-5)
    for p in bufs:
        dp().host_free(p)
