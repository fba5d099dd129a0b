"""Cost of a dependency wait before every loaded unit on the execution stream (all of them
already satisfied), measured on the warm forward: DP_DEBUG_WARM_WAITS = 0 none, 1 event wait,
2 one-thread acquire-spin kernel, 3 cuStreamWaitValue32.  Each setting runs in its own process
(the library reads the variable once).  python tools/wait_cost.py [model:seq]"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
spec = sys.argv[1] if len(sys.argv) > 1 else "bert_base:128"
CHILD = r'''
import json, os, sys
sys.path.insert(0, ROOT)
import numpy as np, torch
import paper_conf_eurosys_jeongba23_b200 as dp, synth
name, S = SPEC.split(":"); S = int(S)
m = synth.SHAPES[name]
ctx = dp.Context([0]); model = dp.Model(ctx, m, synth.make_weights(m, seed=0))
ids = torch.from_numpy(synth.make_ids(m, 1, S)).cuda()
out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
model.infer_cold(dp._lib.PlanArrays(model.n, np.zeros(model.n, np.int8), None, 1, 1), 0, ids, out, pool)
torch.cuda.synchronize()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
res = {}
for graph in (1, 0):
    ctx.set_opts(use_graph=graph)
    ts = []
    for i in range(35):
        flush.fill_(i)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(); model.infer_warm(0, ids, out, pool); e1.record()
        torch.cuda.synchronize()
        if i >= 5: ts.append(e0.elapsed_time(e1))
    res["graph" if graph else "eager"] = round(float(np.median(ts)), 4)
print(json.dumps(res))
'''.replace("ROOT", repr(ROOT)).replace("SPEC", repr(spec))
for mode in (0, 1, 2, 3):
    env = dict(os.environ, DP_DEBUG_WARM_WAITS=str(mode))
    r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True, timeout=600)
    line = r.stdout.strip().splitlines()[-1] if r.returncode == 0 else json.dumps({"error": r.stderr[-500:]})
    print(json.dumps({"model": spec, "waits": ["none", "event", "spin_kernel", "stream_wait_value"][mode],
                      **json.loads(line)}), flush=True)
