"""Fig. 12 on one B200: cold-start throughput vs batch size 1..8 per engine
option, normalised to BASELINE at batch 1 ("We normalize the throughput to Baseline
with batch size 1").  For every (model, batch, mode): a live profile at that batch -> plan ->
cold starts replayed from a CUDA graph (evict + 256 MiB L2 flush between runs, CUDA events on
the execution stream, median of N).  Throughput = batch / cold-start latency.  PT needs more
than one GPU and is not run here.

python tools/batch_sweep.py [model:seq ...]   (default bert_base:128 roberta_large:384 gpt2_medium:1024)
One JSON line per point, then one summary line.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

specs = sys.argv[1:] or ["bert_base:128", "roberta_large:384", "gpt2_medium:1024"]
N = int(os.environ.get("DP_N", "10"))
BATCHES = [int(b) for b in os.environ.get("DP_BATCHES", "1,2,4,8").split(",")]
MODES = os.environ.get("DP_MODES", "BASELINE,PIPESWITCH,DHA,DHA_LINK").split(",")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ctx = dp.Context([0])
ctx.set_opts(use_graph=True)
summary = {}
for spec in specs:
    name, S = spec.split(":")[0], int(spec.split(":")[1])
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=0)
    model = dp.Model(ctx, m, w)
    base = None
    for B in BATCHES:
        ids = torch.from_numpy(synth.make_ids(m, B, S, seed=1)).cuda()
        out = torch.empty(B * S, m.hidden, dtype=torch.float16, device="cuda")
        pool = torch.empty(B, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
        cost = model.profile(0, B, S, 5)
        s = torch.cuda.Stream()
        for mode in MODES:
            plan = dp.plan_generate(cost, mode, 1)
            ts = []
            for i in range(N + 3):
                if model.is_resident(0):
                    model.evict(0)
                flush.fill_(i & 0xFF)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                with torch.cuda.stream(s):
                    e0.record(s)
                    model.infer_cold(plan, 0, ids, out, pool, stream=s)
                    e1.record(s)
                torch.cuda.synchronize()
                if i >= 3:
                    ts.append(e0.elapsed_time(e1))
            model.evict(0)
            ms = float(np.median(ts))
            thr = B / ms * 1e3
            if B == BATCHES[0] and mode == "BASELINE":
                base = thr
            row = {"model": name, "seq": S, "batch": B, "mode": mode, "cold_ms": round(ms, 4),
                   "throughput_per_s": round(thr, 1), "normalised": round(thr / base, 3) if base else None,
                   "dha_units": int(plan.method.sum()),
                   "predicted_ms": round(dp.plan_simulate(cost, plan)[0] / 1e6, 4)}
            summary.setdefault(name, {}).setdefault(mode, {})[B] = row["normalised"]
            print(json.dumps(row), flush=True)
    model.close()
print(json.dumps({"summary_normalised_to_baseline_b1": summary}))
ctx.close()
