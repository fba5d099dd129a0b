"""Diagnostics on the GPU box: per-unit cost table, warm latency by plan, cold latency by
engine options.  python tools/diag.py [model] [seq]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

name = sys.argv[1] if len(sys.argv) > 1 else "bert_base"
S = int(sys.argv[2]) if len(sys.argv) > 2 else 128
m = synth.SHAPES[name]
w = synth.make_weights(m, seed=0)
ctx = dp.Context([0])
ctx.set_opts(use_graph=int(os.environ.get("DP_GRAPH", "1")), use_pdl=int(os.environ.get("DP_PDL", "1")))
model = dp.Model(ctx, m, w)
cost = model.profile(0, 1, S, 10)
units = model.units()
rows = []
for i, u in enumerate(units):
    rows.append({k: int(cost[k][i]) for k in cost} | {"name": u["name"]})
ids = torch.from_numpy(synth.make_ids(m, 1, S)).cuda()
out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
res = {"model": name, "seq": S, "cost": rows}


def timed(fn, n=10):
    ts = []
    for _ in range(n):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


for mode in ("PIPESWITCH", "GREEDY", "DHA", "BASELINE"):
    plan = dp.plan_generate(cost, mode, 1)
    pred = dp.plan_simulate(cost, plan)[0] / 1e6

    def cold():
        if model.is_resident(0):
            model.evict(0)
        model.infer_cold(plan, 0, ids, out, pool)
    c = timed(cold)
    w_ms = timed(lambda: model.infer_warm(0, ids, out, pool))
    model.evict(0)
    res[mode] = {"cold_ms": c, "warm_ms": w_ms, "pred_ms": pred, "dha_units": int(plan.method.sum()),
                 "dha_names": [units[i]["name"] for i in range(len(units)) if plan.method[i]][:50]}
plan = dp.plan_generate(cost, "DHA", 1)
for chunk in (1, 2, 4, 8, 16, 64):
    for ns in (1, 2, 3):
        ctx.set_opts(chunk_bytes=chunk << 20, n_h2d_streams=ns)

        def cold():
            if model.is_resident(0):
                model.evict(0)
            model.infer_cold(plan, 0, ids, out, pool)
        res[f"cold_chunk{chunk}MB_s{ns}"] = timed(cold)
print(json.dumps(res))
