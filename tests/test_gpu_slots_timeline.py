"""HBM slots from the per-device pool, LOAD-only layout, and the per-unit timeline (GPU).

* P:332 ("DeepPlan can serve more instances"): a resident model holds HBM only for its LOADED
  units -- the slot block is the arena layout with every DHA unit's range left out; outputs are
  unchanged (the same kernels read the same bytes);
* dp_model_evict returns the block to the context's pool: the next cold start (of the same or
  another model) reuses it, dp_pool_trim gives free blocks back to the driver;
* SURVEY §8(b) per-unit ready/start/end ns (dp_run_timeline, opts.trace_units): every loaded
  unit's first kernel starts after its bytes landed (the event gate of P:235, observed), the
  measured stalls track the pipeline simulator's on a live profile.
"""
import numpy as np
import pytest

import synth
from oracle import forward as F
from oracle import planner as OP

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def run_cold(model, plan, ids_np):
    B, S = ids_np.shape
    ids = torch.from_numpy(ids_np).cuda()
    out = torch.empty(B * S, model.shape.hidden, dtype=torch.float16, device="cuda")
    pool = torch.empty(B, model.shape.hidden, dtype=torch.float16, device="cuda") \
        if model.shape.family != "gpt2" else None
    st = model.infer_cold(plan, 0, ids, out, pool)
    torch.cuda.synchronize()
    return out, pool, st


def arena_spans(model):
    us = model.units()
    total = len(model.arena())  # arena bytes incl. alignment padding
    return [(us[i + 1]["offset"] if i + 1 < len(us) else total) - us[i]["offset"] for i in range(len(us))]


@pytest.mark.parametrize("name", ["tiny_bert", "bert_base", "tiny_gpt2"])
def test_resident_bytes_are_the_loaded_units_only(name):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=1, dtype="fp16")
    ids = synth.make_ids(m, 1, 64, seed=2)
    c = dp().Context([0])
    c.set_opts(debug_poison=1)
    model = dp().Model(c, m, w, "fp16")
    n = model.n
    kinds = [u["kind"] for u in model.units()]
    spans = arena_spans(model)
    all_load = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1)
    # embeddings + every LayerNorm by DHA (the word table is the big one)
    meth = np.array([1 if k in ("emb", "ln") else 0 for k in kinds], np.int8)
    emb_dha = dp()._lib.PlanArrays(n, meth, None, 3, 1)
    a, pa, _ = run_cold(model, all_load, ids)
    full = model.resident_bytes(0)
    assert full == len(model.arena())
    a = a.clone()
    model.evict(0)
    assert model.resident_bytes(0) == 0
    b, pb, st = run_cold(model, emb_dha, ids)
    dha_span = sum(s for s, k in zip(spans, meth) if k)
    want = len(model.arena()) - dha_span
    got = model.resident_bytes(0)
    assert got == want, (got, want)  # exactly the loaded units' ranges (with their alignment)
    assert torch.equal(a, b)         # same outputs from the compact layout
    # the DMA carried exactly the loaded units, into the compact block
    assert st["h2d_bytes"][0] == sum(u["bytes"] for u, k in zip(model.units(), meth) if not k)
    model.evict(0)
    model.close()
    c.close()


def test_evict_returns_the_block_to_the_pool_and_trim_frees_it():
    m = synth.SHAPES["bert_base"]
    w = synth.make_weights(m, seed=3, dtype="fp16")
    ids = synth.make_ids(m, 1, 128, seed=4)
    c = dp().Context([0])
    c.set_opts(use_graph=1)
    m1 = dp().Model(c, m, w, "fp16")
    m2 = m1.clone()
    n = m1.n
    plan = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1)
    o1, _, _ = run_cold(m1, plan, ids)
    r0, u0 = c.pool_stats(0)
    assert u0 == r0 >= m1.nbytes
    o1 = o1.clone()
    m1.evict(0)
    r1, u1 = c.pool_stats(0)
    assert (r1, u1) == (r0, 0)  # back to the pool, not to the driver
    o2, _, _ = run_cold(m2, plan, ids)  # another instance reuses the block
    assert c.pool_stats(0) == (r0, r0)
    assert torch.equal(o1, o2)
    # both resident: a second block
    o3, _, _ = run_cold(m1, plan, ids)
    r3, u3 = c.pool_stats(0)
    assert r3 == 2 * r0 and u3 == r3 and torch.equal(o3, o1)
    m1.evict(0)
    m2.evict(0)
    assert c.pool_trim(0) == 2 * r0
    assert c.pool_stats(0) == (0, 0)
    # graph replay after the pool handed out new blocks is still correct
    for _ in range(2):
        o4, _, _ = run_cold(m1, plan, ids)
        assert torch.equal(o4, o1)
        m1.evict(0)
    m1.close()
    m2.close()
    c.close()


@pytest.mark.parametrize("mode", ["PIPESWITCH", "DHA", "DHA_LINK"])
def test_timeline_gates_and_tracks_the_simulator(mode):
    m = synth.SHAPES["bert_base"]
    w = synth.make_weights(m, seed=5, dtype="fp16")
    ids = synth.make_ids(m, 1, 128, seed=6)
    c = dp().Context([0])
    model = dp().Model(c, m, w, "fp16")
    cost = model.profile(0, 1, 128, iters=5)
    plan = dp().plan_generate(cost, mode, 1)
    c.set_opts(trace_units=1, debug_poison=1)
    out, pool, _ = run_cold(model, plan, ids)
    tl = model.timeline(0)
    ref, ref_pool = F.forward(m, w, ids, "fp16")
    assert np.abs(out.double().cpu().numpy() - ref.reshape(128, -1)).max() <= 1e-2  # tracing changes nothing
    model.evict(0)
    ready, start, end, stall = tl["ready_ns"], tl["start_ns"], tl["end_ns"], tl["stall_ns"]
    meth = np.array(plan.method)
    assert np.all(start >= 0) and np.all(end >= start)  # every unit reached (pooler too)
    loaded = meth == 0
    # P:235 observed: a loaded unit's kernels start only after its bytes landed
    assert np.all(start[loaded] >= ready[loaded] - 2000), (start - ready)[loaded].min()
    assert np.all(ready[~loaded] == 0)
    # one link: pieces land in order
    r = ready[loaded]
    assert np.all(np.diff(r) >= 0)
    # the pipeline recurrence of P:162-170 holds on the hardware: a unit starts when
    # the stream reached it or when its bytes landed, whichever is later, so its stall is
    # max(0, ready - reached) -- up to the timestamp kernels' own launch (a few us) and the event
    # wait's latency
    pre = start - stall
    want = np.where(loaded, np.maximum(0, ready - pre), 0)
    assert np.all(np.abs(stall - want) <= 30_000), np.abs(stall - want).max()
    # against the simulator on the same live profile (R23 calibration).  Tracing puts two events
    # around every unit (no PDL overlap), which slows the compute chain and hides some stall, so
    # the comparison is loose; the paper-model DHA plan is known to under-predict (it ignores
    # the DHA reads' share of the link, G11 / R19) and is not compared
    lat, sim_stall, _ = dp().plan_simulate(cost, plan)
    if mode != "DHA":
        assert abs(end.max() - lat) <= 0.35 * lat, (end.max(), lat)
    if mode == "PIPESWITCH":  # load-bound: the stalls dominate and must match
        meas_total, sim_total = float(stall.sum()), float(sim_stall.sum())
        assert abs(meas_total - sim_total) <= 0.3 * sim_total + 300_000, (meas_total, sim_total)
    model.close()
    c.close()


def test_timeline_needs_a_traced_run():
    m = synth.SHAPES["tiny_bert"]
    w = synth.make_weights(m, seed=7, dtype="fp16")
    c = dp().Context([0])
    model = dp().Model(c, m, w, "fp16")
    with pytest.raises(dp().DeepPlanError):
        model.timeline(0)
    model.close()
    c.close()


def test_failed_cold_start_returns_the_block():
    """A cold start that fails after taking its HBM block (here: a PT secondary outside the context)
    hands the block back: nothing is held and the next cold start works."""
    m = synth.SHAPES["tiny_bert"]
    w = synth.make_weights(m, seed=9, dtype="fp16")
    ids = synth.make_ids(m, 1, 32, seed=10)
    c = dp().Context([0])
    model = dp().Model(c, m, w, "fp16")
    n = model.n
    pt = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), np.array([i % 2 for i in range(n)], np.int8), 4, 2)
    out = torch.empty(32, m.hidden, dtype=torch.float16, device="cuda")
    with pytest.raises(dp().DeepPlanError):
        model.infer_cold(pt, 0, torch.from_numpy(ids).cuda(), out, secondaries=[5])
    assert not model.is_resident(0) and c.pool_stats(0)[1] == 0
    ok = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1)
    run_cold(model, ok, ids)
    assert model.is_resident(0)
    model.evict(0)
    model.close()
    c.close()
