"""Multi-instance serving on real GPUs (§5.3).

Instances are clones of registered base models (same shapes, shared pinned arena, separate
residency), mixed by ratio (BERT-Base : RoBERTa-Base : GPT-2 = 4:4:1).  Each plan mode
(PIPESWITCH = all loaded, DHA = Algorithm 1, DHA_LINK, PT_DHA* with several GPUs) gets its
measured cold / warm latency and resident bytes per model (DHA units stay in host memory,
P:332); a seeded Poisson trace is served live through dp_serve_run -- the online
dispatcher (one request per GPU at a time, real LRU evictions under a per-GPU budget, PT
secondaries borrowed from idle GPUs) -- beside the dry-run replay with the measured latency
table (tests/test_gpu_serving.py checks the live decisions against the oracle's re-derivation).  Reports p99, goodput at the SLO,
the cold-start rate and throughput, beside the dry-run replay of the same decisions.

python tools/serve_bench.py [--gpus 1] [--mix bert_base:128:1] [--instances 40] [--fit 8]
                            [--rate 300] [--requests 600] [--slo-ms 10] [--modes PIPESWITCH,DHA,DHA_LINK]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth


def dev_ms(fn, reps=6):
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts[1:]))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--mix", default="bert_base:128:1", help="name:seq:weight,...")
    ap.add_argument("--instances", type=int, default=40)
    ap.add_argument("--fit", type=float, default=8, help="all-loaded instances of model 0 per GPU budget")
    ap.add_argument("--rate", type=float, default=300.0, help="requests per second (Poisson)")
    ap.add_argument("--requests", type=int, default=600)
    ap.add_argument("--slo-ms", type=float, default=10.0)
    ap.add_argument("--modes", default="PIPESWITCH,DHA,DHA_LINK")
    ap.add_argument("--trace", default="poisson", choices=["poisson", "maf"],
                    help="poisson (P:328) or the synthetic MAF-like bursty trace (P:342-350, SURVEY f2)")
    ap.add_argument("--duration", type=float, default=20.0, help="maf: trace seconds (rate x duration requests)")
    ap.add_argument("--window", type=float, default=1.0, help="maf: seconds per timeline window (Fig. 15)")
    a = ap.parse_args()
    mix = [(n, int(s), int(wt)) for n, s, wt in (x.split(":") for x in a.mix.split(","))]
    ctx = dp.Context(list(range(a.gpus)))
    ctx.set_opts(use_graph=1)
    bases, costs, io = [], [], []
    for name, seq, _ in mix:
        m = synth.SHAPES[name]
        base = dp.Model(ctx, m, synth.make_weights(m, seed=0))
        costs.append(base.profile(0, 1, seq, 5))
        bases.append(base)
        ids = torch.from_numpy(synth.make_ids(m, 1, seq)).cuda()
        out = torch.empty(seq, m.hidden, dtype=torch.float16, device="cuda")
        pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
        io.append((ids, out, pool))
    moi = synth.instance_models(a.instances, tuple(w for _, _, w in mix)) if len(mix) > 1 \
        else np.zeros(a.instances, np.int32)
    insts = [bases[moi[i]].clone() for i in range(a.instances)]  # the bases are profiling-only
    budget = int(a.fit * bases[0].nbytes)
    if a.trace == "maf":
        arr, inst = synth.make_maf_like_trace(a.duration, a.rate, a.instances, seed=11)
        a.requests = len(arr)
    else:
        arr, inst = synth.make_poisson_trace(a.requests, a.rate, a.instances, seed=11)
    report = {"trace": a.trace, "mix": a.mix, "gpus": a.gpus, "instances": a.instances, "rate_rps": a.rate, "requests": a.requests,
              "slo_ms": a.slo_ms, "per_gpu_budget_bytes": budget, "modes": {}}
    for mode in a.modes.split(","):
        k = a.gpus if mode.startswith("PT") else 1
        plans, cold, warm, resident = [], [], [], []
        for mi, base in enumerate(bases):
            plan = dp.plan_generate(costs[mi], mode, k)
            sec = list(range(1, k))
            ids, out, pool = io[mi]

            def cold_run():
                if base.is_resident(0):
                    base.evict(0)
                base.infer_cold(plan, 0, ids, out, pool, secondaries=sec)
            cold.append(int(dev_ms(cold_run) * 1e6))
            warm.append(int(dev_ms(lambda: base.infer_warm(0, ids, out, pool)) * 1e6))
            base.evict(0)
            plans.append(plan)
            resident.append(dp.plan_resident_bytes(base, plan))  # the compact slot block (loaded units)
        kw = dict(ngpu=a.gpus, per_gpu_budget_bytes=budget, cold_ns=cold, warm_ns=warm, resident_bytes=resident,
                  model_of_instance=moi, slo_ns=int(a.slo_ms * 1e6), batch=1,
                  seq=max(s for _, s, _ in mix), seq_of_model=[s for _, s, _ in mix])
        dry = dp.serve_run(arr, inst, dry_run=True, **kw)
        live = dp.serve_run(arr, inst, dry_run=False, ctx=ctx, models=insts,
                            plans=[plans[moi[i]] for i in range(a.instances)], **kw)

        for i in insts + bases:
            for g in range(a.gpus):
                if i.is_resident(g):
                    i.evict(g)

        def summarize(r, timeline=False):
            lat = (r["finish_ns"] - arr) / 1e6
            out = {"p99_ms": round(float(np.percentile(lat, 99)), 3), "p50_ms": round(float(np.median(lat)), 3),
                   "goodput": round(float(np.mean(lat <= a.slo_ms)), 4),
                   "cold_rate": round(float(np.mean(r["cold"])), 4),
                   "throughput_rps": round(len(lat) / ((r["finish_ns"].max() - arr.min()) / 1e9), 1)}
            if timeline and a.trace == "maf":  # Fig. 15: offered load and p99 / goodput per window
                w = (arr // int(a.window * 1e9)).astype(np.int64)
                out["timeline"] = [{"t_s": int(k * a.window), "offered_rps": round(float(np.sum(w == k)) / a.window, 1),
                                    "p99_ms": round(float(np.percentile(lat[w == k], 99)), 3),
                                    "goodput": round(float(np.mean(lat[w == k] <= a.slo_ms)), 4),
                                    "cold_rate": round(float(np.mean(r["cold"][w == k])), 4)}
                                   for k in np.unique(w)]
            return out
        report["modes"][mode] = {
            "per_model": {mix[mi][0]: {"cold_ms": cold[mi] / 1e6, "warm_ms": warm[mi] / 1e6,
                                       "resident_mb": round(resident[mi] / 2 ** 20, 1),
                                       "dha_units": int(plans[mi].method.sum())} for mi in range(len(mix))},
            "live": summarize(live, timeline=True), "replay": summarize(dry),
            "pt_cold_starts_with_secondaries": int(np.sum((live["cold"] == 1) & (live["sec_mask"] != 0)))}
    print(json.dumps(report))


if __name__ == "__main__":
    main()
