"""Planner comparison on real profiles (Table 3, Fig.11 analogue).

For each model: profile on this GPU (dp_profile), then for every engine option and
k in {1, 2, 4, 8}: the plan, its simulated latency (the paper's model and the link-aware
model), and -- for k = 1, the only thing one GPU can run -- the measured cold-start
latency.  A windowed exhaustive search (first `--window` units exhaustive, the rest fixed
to Algorithm 1's choice) bounds how far Algorithm 1 is from the model's optimum.

python tools/plan_compare.py [bert_large:384 gpt2_medium:1024 roberta_large:384 bert_base:128]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

specs = sys.argv[1:] or ["bert_base:128", "bert_large:384", "roberta_large:384", "gpt2_medium:1024"]
window = int(os.environ.get("DP_WINDOW", "16"))
ctx = dp.Context([0])
ctx.set_opts(use_graph=1)
report = {}
for spec in specs:
    name, S = spec.split(":")
    S = int(S)
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=0)
    model = dp.Model(ctx, m, w)
    t0 = time.perf_counter()
    cost = model.profile(0, 1, S, 10)
    prof_s = time.perf_counter() - t0
    ids = torch.from_numpy(synth.make_ids(m, 1, S)).cuda()
    out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
    pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
    res = {"units": model.n, "bytes": int(model.nbytes), "profile_s": round(prof_s, 2), "plans": {}}
    for mode in ("BASELINE", "PIPESWITCH", "GREEDY", "DHA", "DHA_LINK", "PT", "PT_DHA", "PT_DHA_LINK", "PT_DHA_BAL", "PT_DHA_LINK_BAL",
                 "PT_DHA_STRIPE", "PT_DHA_LINK_STRIPE"):
        for k in ((1, 2, 4, 8) if mode.startswith("PT") else (1,)):
            plan = dp.plan_generate(cost, mode, k)
            lat, _, link = dp.plan_simulate(cost, plan)
            entry = {"dha_units": int(plan.method.sum()), "sim_ms": round(lat / 1e6, 4),
                     "link_mb": [round(x / 2 ** 20, 1) for x in link]}
            if k == 1:
                ts = []
                for i in range(8):
                    if model.is_resident(0):
                        model.evict(0)
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    model.infer_cold(plan, 0, ids, out, pool)
                    e1.record()
                    torch.cuda.synchronize()
                    if i >= 2:
                        ts.append(e0.elapsed_time(e1))
                entry["measured_ms"] = round(float(np.mean(ts)), 4)
            res["plans"][f"{mode}/k{k}"] = entry
    if model.is_resident(0):
        model.evict(0)
    # windowed exhaustive (paper model), k = 1 and 8
    for k in (1, 8):
        base = dp.plan_generate(cost, "PT_DHA" if k > 1 else "DHA", k)
        part = dp.plan_partition(cost["bytes"], k) if k > 1 else np.zeros(model.n, np.int8)
        free = [i for i in range(model.n) if part[i] == 0][:window]
        t0 = time.perf_counter()
        lat, p = dp.plan_exhaustive(cost, base, free)
        res["plans"][f"EXHAUSTIVE_w{len(free)}/k{k}"] = {"sim_ms": round(lat / 1e6, 4),
                                                      "dha_units": int(p.method.sum()),
                                                      "search_s": round(time.perf_counter() - t0, 2)}
    # windowed exhaustive over the striped split (R22) at k = 8: the first `window` slot-0
    # units free (the striped plan's own partition kept)
    base = dp.plan_generate(cost, "PT_DHA_STRIPE", 8)
    free = [i for i in range(model.n) if base.slot[i] == 0][:window]
    t0 = time.perf_counter()
    lat, p = dp.plan_exhaustive(cost, base, free)
    res["plans"][f"EXHAUSTIVE_STRIPE_w{len(free)}/k8"] = {"sim_ms": round(lat / 1e6, 4),
                                                         "dha_units": int(p.method.sum()),
                                                         "search_s": round(time.perf_counter() - t0, 2)}
    model.close()
    report[spec] = res
print(json.dumps(report, indent=1))
