"""Fig. 2 on B200: where a cold start's time goes, measured per unit.

For each model and engine option: a live profile, the plan, one cold start with
opts.trace_units (dp_run_timeline: per-unit ready / start / end / stall ns), and the totals --
latency, the execution stream's stall (waiting for weights), the compute time -- beside the
pipeline simulator's prediction.  The paper measured 73-75% of PipeSwitch's latency as stall for
BERT / RoBERTa on V100.  Tracing launches two timestamp kernels per unit (a few us each, no PDL
overlap between units), so the traced latency is a little above the untraced one.

python tools/stall_breakdown.py [model:seq ...] [--modes PIPESWITCH,DHA,DHA_LINK] [--out FILE]
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
    ap.add_argument("cases", nargs="*", default=["bert_base:128", "roberta_large:384", "gpt2_medium:1024"])
    ap.add_argument("--modes", default="PIPESWITCH,DHA,DHA_LINK")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    rows = []
    for case in a.cases:
        name, S = case.split(":")
        S = int(S)
        m = synth.SHAPES[name]
        ctx = dp.Context([0])
        model = dp.Model(ctx, m, synth.make_weights(m, seed=0))
        cost = model.profile(0, 1, S, 5)
        ids = torch.from_numpy(synth.make_ids(m, 1, S, seed=1)).cuda()
        out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
        pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
        flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
        for mode in a.modes.split(","):
            plan = dp.plan_generate(cost, mode, 1)
            lat_sim, stall_sim, _ = dp.plan_simulate(cost, plan)
            ctx.set_opts(trace_units=1)
            best = None
            for rep in range(3):
                flush.fill_(rep)
                torch.cuda.synchronize()
                model.infer_cold(plan, 0, ids, out, pool)
                tl = model.timeline(0)
                model.evict(0)
                lat = int(tl["end_ns"].max())
                if best is None or lat < best[0]:
                    best = (lat, tl)
            ctx.set_opts(trace_units=0)
            lat, tl = best
            stall = int(tl["stall_ns"][tl["stall_ns"] >= 0].sum())
            row = {"model": name, "seq": S, "mode": mode, "dha_units": int(plan.method.sum()),
                   "latency_ms": round(lat / 1e6, 4), "stall_ms": round(stall / 1e6, 4),
                   "stall_share": round(stall / lat, 4), "compute_ms": round((lat - stall) / 1e6, 4),
                   "simulated_latency_ms": round(lat_sim / 1e6, 4),
                   "simulated_stall_share": round(float(np.sum(stall_sim)) / lat_sim, 4),
                   "largest_stalls": [{"unit": model.units()[int(u)]["name"], "ms": round(int(tl["stall_ns"][u]) / 1e6, 4)}
                                      for u in np.argsort(-tl["stall_ns"])[:5]]}
            rows.append(row)
            print(json.dumps(row), flush=True)
        model.close()
        ctx.close()
    if a.out:
        with open(a.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
