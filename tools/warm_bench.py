"""Warm-forward latency (all units resident) of the per-kernel PDL-chained path, CUDA
graph replay, CUDA events on the launching stream, median of N after warm-up; L2 flushed
between runs (256 MiB write) unless DP_NO_FLUSH=1.  DP_ATT_TC sets opts.attention_tc (0 by sequence
length -- the default --, 1 always K5t, 2 never); the output is compared with the mma.sync path's.

python tools/warm_bench.py [model:seq[:batch] ...]   (default bert_base:128 bert_large:384 gpt2:256)
Prints one JSON line per (model, path).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

specs = sys.argv[1:] or ["bert_base:128", "bert_large:384", "gpt2:256"]
N = int(os.environ.get("DP_N", "30"))
flush = None if os.environ.get("DP_NO_FLUSH") else torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ctx = dp.Context([0])
for spec in specs:
    parts = spec.split(":")
    name, S = parts[0], int(parts[1])
    B = int(parts[2]) if len(parts) > 2 else 1
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=0)
    model = dp.Model(ctx, m, w)
    n = model.n
    ids = torch.from_numpy(synth.make_ids(m, B, S)).cuda()
    out = torch.empty(B * S, m.hidden, dtype=torch.float16, device="cuda")
    pool = torch.empty(B, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
    plan = dp._lib.PlanArrays(n, np.zeros(n, np.int8), np.zeros(n, np.int8), 1, 1)
    ctx.set_opts(attention_tc=2)  # the reference output: the mma.sync attention
    model.infer_cold(plan, 0, ids, out, pool)
    torch.cuda.synchronize()
    ref = out.clone()
    for path in ("per_kernel",):  # (the fused-LN and K6 persistent paths: tools/experiments)
        att_tc = int(os.environ.get("DP_ATT_TC", "0"))
        ctx.set_opts(use_graph=True, attention_tc=att_tc)
        s = torch.cuda.current_stream()
        ts = []
        for i in range(N + 5):
            if flush is not None:
                flush.fill_(i & 0xFF)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(s)
            st = model.infer_warm(0, ids, out, pool)
            e1.record(s)
            torch.cuda.synchronize()
            if i >= 5:
                ts.append(e0.elapsed_time(e1))
        diff = float((out.float() - ref.float()).abs().max())
        print(json.dumps({"model": name, "seq": S, "batch": B, "path": path, "attention_tc": att_tc, "warm_ms_median": round(float(np.median(ts)), 4),
                          "warm_ms_min": round(float(np.min(ts)), 4), "kernels": st["n_kernels"],
                          "max_abs_diff_vs_per_kernel": diff, "l2_flushed": flush is not None}), flush=True)
    model.close()
ctx.close()
