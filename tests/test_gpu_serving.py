"""Live multi-instance serving on the GPU.

dp_serve_run(dry_run=0) is an online dispatcher on the GPUs' observed state (serve_live.cu):
* its decisions (GPU, cold / warm, evictions) equal the oracle's re-derivation of the live policy
  from what the dispatcher had observed when deciding (oracle/serving.py replay_online);
* evictions are real: after the run the device's slot pool holds exactly the resident
  instances' blocks (HBM returned on eviction), and the still-resident instances compute the
  oracle's outputs (sampled with warm inferences on the serving token ids);
* with DHA the instances hold only their loaded units, so more of them fit the same
  per-GPU budget and fewer requests need a cold start than with every unit loaded (PipeSwitch).
"""
import numpy as np
import pytest

import synth
from oracle import forward as F
from oracle import serving as OS
from oracle import units as OU

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def serving_ids(seq):
    return np.array([[3 + (t * 7919) % 997 for t in range(seq)]], dtype=np.int32)


def plans_for(models, mode):
    n = models[0].n
    if mode == "PIPESWITCH":
        meth = np.zeros(n, np.int8)
    else:  # embeddings by DHA (what Algorithm 1 picks on B200 for BERT: the word table)
        kinds = [u["kind"] for u in models[0].units()]
        meth = np.array([1 if k == "emb" else 0 for k in kinds], np.int8)
    return [dp()._lib.PlanArrays(n, meth, None, 1, 1) for _ in models]


def run_live(ctx, models, plans, arr, inst, budget, ngpu=1, seq=32):
    n_inst = len(models)
    return dp().serve_run(arr, inst, ngpu=ngpu, per_gpu_budget_bytes=budget, cold_ns=[1], warm_ns=[1],
                          resident_bytes=[1], model_of_instance=np.zeros(n_inst, np.int32), dry_run=False, ctx=ctx,
                          models=models, plans=plans, batch=1, seq=seq)


@pytest.mark.parametrize("name,seq", [("tiny_bert", 32), ("tiny_gpt2", 48)])
def test_live_decisions_equal_oracle_replay_and_evictions_free_hbm(name, seq):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=1, dtype="fp16")
    c = dp().Context([0])
    c.set_opts(use_graph=1)
    base = dp().Model(c, m, w, "fp16")
    models = [base.clone() for _ in range(8)]
    plans = plans_for(models, "DHA")
    rb = [dp().plan_resident_bytes(mm, p) for mm, p in zip(models, plans)]
    budget = int(3.5 * rb[0])
    arr, inst = synth.make_poisson_trace(300, 400.0, len(models), seed=5)
    res = run_live(c, models, plans, arr, inst, budget, seq=seq)
    ref = OS.replay_online(arr, inst, ngpu=1, per_gpu_budget_bytes=budget, resident_bytes=rb,
                           decide_ns=res["decide_ns"], finish_ns=res["finish_ns"])
    for k in ("gpu", "cold", "nevicted"):
        assert np.array_equal(res[k], ref[k]), k
    assert np.all(res["decide_ns"] >= arr) and np.all(res["start_ns"] >= res["decide_ns"])
    assert np.all(res["finish_ns"] > res["start_ns"])
    assert 0 < res["cold"].sum() < len(arr) and res["nevicted"].sum() > 0
    # real eviction: exactly the instances the policy left resident are resident (the GPU may run
    # over budget while every resident instance still has work, R11-live), and the pool holds
    # exactly their blocks
    resident = [mm for mm in models if mm.is_resident(0)]
    assert [i for i, mm in enumerate(models) if mm.is_resident(0)] == ref["resident"][0]
    _, in_use = c.pool_stats(0)
    grain = 2 << 20
    assert in_use == sum(-(-mm.resident_bytes(0) // grain) * grain for mm in resident)
    # the resident instances' weights are right: warm inferences vs the oracle
    ids = serving_ids(seq)
    refo, _ = F.forward(m, w, ids, "fp16")
    for mm in resident:
        out = torch.empty(seq, m.hidden, dtype=torch.float16, device="cuda")
        pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
        mm.infer_warm(0, torch.from_numpy(ids).cuda(), out, pool)
        torch.cuda.synchronize()
        assert np.abs(out.double().cpu().numpy() - refo.reshape(seq, -1)).max() <= 1e-2
    for mm in models:
        if mm.is_resident(0):
            mm.evict(0)
        mm.close()
    base.close()
    c.close()


def test_dha_fits_more_instances_than_pipeswitch():
    """DHA keeps the embedding tables in host memory, so under the same per-GPU budget more
    instances stay resident and fewer requests pay a cold start."""
    m = synth.SHAPES["tiny_bert"]
    w = synth.make_weights(m, seed=2, dtype="fp16")
    c = dp().Context([0])
    c.set_opts(use_graph=1)
    base = dp().Model(c, m, w, "fp16")
    models = [base.clone() for _ in range(8)]
    full = dp().plan_resident_bytes(models[0], plans_for(models, "PIPESWITCH")[0])
    budget = int(3.3 * full)
    arr, inst = synth.make_poisson_trace(400, 800.0, len(models), seed=9)
    cold = {}
    for mode in ("PIPESWITCH", "DHA"):
        plans = plans_for(models, mode)
        res = run_live(c, models, plans, arr, inst, budget)
        cold[mode] = int(res["cold"].sum())
        fits = budget // dp().plan_resident_bytes(models[0], plans[0])
        assert fits == (3 if mode == "PIPESWITCH" else 4)
        for mm in models:
            if mm.is_resident(0):
                mm.evict(0)
    assert cold["DHA"] < cold["PIPESWITCH"], cold
    for mm in models:
        mm.close()
    base.close()
    c.close()


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2, reason="needs >= 2 GPUs")
def test_live_pt_cold_starts_borrow_idle_gpus():
    """Two GPUs: PT cold starts (k = 2) borrow the other GPU's link; decisions = the replay."""
    m = synth.SHAPES["bert_base"]
    w = synth.make_weights(m, seed=3, dtype="fp16")
    c = dp().Context([0, 1])
    c.set_opts(use_graph=1, pt_transport="ce")
    base = dp().Model(c, m, w, "fp16")
    models = [base.clone() for _ in range(6)]
    n = base.n
    nb = np.array(OU.unit_bytes(m, "fp16"), np.int64)
    slot = np.array([0 if i % 2 == 0 else 1 for i in range(n)], np.int8)
    plans = [dp()._lib.PlanArrays(n, np.zeros(n, np.int8), slot, 4, 2) for _ in models]
    rb = [dp().plan_resident_bytes(mm, p) for mm, p in zip(models, plans)]
    budget = int(2.5 * rb[0])
    arr, inst = synth.make_poisson_trace(200, 500.0, len(models), seed=4)
    res = run_live(c, models, plans, arr, inst, budget, ngpu=2, seq=128)
    ref = OS.replay_online(arr, inst, ngpu=2, per_gpu_budget_bytes=budget, resident_bytes=rb,
                           decide_ns=res["decide_ns"], finish_ns=res["finish_ns"])
    for k in ("gpu", "cold", "nevicted"):
        assert np.array_equal(res[k], ref[k]), k
    colds = res["cold"] == 1
    assert np.all(res["sec_mask"][colds] == np.where(res["gpu"][colds] == 0, 2, 1))
    assert nb.sum() > 0
    for mm in models:
        for d in (0, 1):
            if mm.is_resident(d):
                mm.evict(d)
        mm.close()
    base.close()
    c.close()
