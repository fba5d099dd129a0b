"""Multi-instance serving on real GPUs (§5.3).

Instances are clones of one registered model (same shapes, shared pinned arena, separate
residency).  Each plan mode (PIPESWITCH = all loaded, DHA = Algorithm 1, PT_DHA when several
GPUs) gets its measured cold / warm latency and resident bytes (DHA units stay in host
memory); a seeded Poisson trace is replayed live through dp_serve_run with
one request per GPU at a time and LRU eviction under a per-GPU budget.  Reports p99,
goodput at the SLO and the cold-start rate, beside the dry-run replay of the same decisions.

python tools/serve_bench.py [--gpus 1] [--instances 40] [--fit 8] [--rate 400] [--requests 600]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--model", default="bert_base")
    ap.add_argument("--seq", type=int, default=128)
    ap.add_argument("--instances", type=int, default=40)
    ap.add_argument("--fit", type=int, default=8, help="all-loaded instances that fit one GPU's budget")
    ap.add_argument("--rate", type=float, default=400.0, help="requests per second (Poisson)")
    ap.add_argument("--requests", type=int, default=600)
    ap.add_argument("--slo-ms", type=float, default=10.0)
    ap.add_argument("--modes", default="PIPESWITCH,DHA")
    a = ap.parse_args()
    m = synth.SHAPES[a.model]
    w = synth.make_weights(m, seed=0)
    ctx = dp.Context(list(range(a.gpus)))
    ctx.set_opts(use_graph=1)
    base = dp.Model(ctx, m, w)
    cost = base.profile(0, 1, a.seq, 5)
    insts = [base] + [base.clone() for _ in range(a.instances - 1)]
    ids = torch.from_numpy(synth.make_ids(m, 1, a.seq)).cuda()
    out = torch.empty(a.seq, m.hidden, dtype=torch.float16, device="cuda")
    pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
    budget = a.fit * base.nbytes
    arr, inst = synth.make_poisson_trace(a.requests, a.rate, a.instances, seed=11)
    report = {"model": a.model, "seq": a.seq, "gpus": a.gpus, "instances": a.instances, "rate_rps": a.rate,
              "requests": a.requests, "slo_ms": a.slo_ms, "per_gpu_budget_bytes": budget, "modes": {}}
    for mode in a.modes.split(","):
        k = a.gpus if mode.startswith("PT") else 1
        plan = dp.plan_generate(cost, mode, k)
        sec = list(range(1, k))

        def cold():
            if base.is_resident(0):
                base.evict(0)
            base.infer_cold(plan, 0, ids, out, pool, secondaries=sec)
        times = []
        for _ in range(6):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            if base.is_resident(0):
                base.evict(0)
            torch.cuda.synchronize()
            e0.record()
            base.infer_cold(plan, 0, ids, out, pool, secondaries=sec)
            e1.record()
            torch.cuda.synchronize()
            times.append(e0.elapsed_time(e1))
        cold_ns = int(np.median(times[1:]) * 1e6)
        wt = []
        for _ in range(6):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            base.infer_warm(0, ids, out, pool)
            e1.record()
            torch.cuda.synchronize()
            wt.append(e0.elapsed_time(e1))
        warm_ns = int(np.median(wt[1:]) * 1e6)
        base.evict(0)
        resident = int(sum(b for b, mt in zip(base.unit_bytes(), plan.method) if mt == dp.LOAD))
        kw = dict(ngpu=a.gpus, per_gpu_budget_bytes=budget, cold_ns=[cold_ns], warm_ns=[warm_ns],
                  resident_bytes=[resident], model_of_instance=np.zeros(a.instances, np.int32),
                  slo_ns=int(a.slo_ms * 1e6), batch=1, seq=a.seq)
        dry = dp.serve_run(arr, inst, dry_run=True, **kw)
        live = dp.serve_run(arr, inst, dry_run=False, ctx=ctx, models=insts, plans=[plan] * a.instances, **kw)
        for i in insts:
            for g in range(a.gpus):
                if i.is_resident(g):
                    i.evict(g)

        def summarize(r):
            lat = (r["finish_ns"] - arr) / 1e6
            return {"p99_ms": round(float(np.percentile(lat, 99)), 3), "p50_ms": round(float(np.median(lat)), 3),
                    "goodput": round(float(np.mean(lat <= a.slo_ms)), 4),
                    "cold_rate": round(float(np.mean(r["cold"])), 4),
                    "throughput_rps": round(len(lat) / ((r["finish_ns"].max() - arr.min()) / 1e9), 1)}
        report["modes"][mode] = {"cold_ms": cold_ns / 1e6, "warm_ms": warm_ns / 1e6, "resident_mb": resident / 2**20,
                                 "instances_fit_per_gpu": budget // resident, "live": summarize(live),
                                 "replay": summarize(dry)}
    print(json.dumps(report))


if __name__ == "__main__":
    main()
