import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_eurosys_jeongba23_b200 as dp, synth
m = synth.SHAPES["tiny_bert"]; w = synth.make_weights(m, seed=2)
c = dp.Context([0]); c.set_opts(use_graph=1)
base = dp.Model(c, m, w); models = [base.clone() for _ in range(8)]
n = base.n
kinds = [u["kind"] for u in base.units()]
plans = [dp._lib.PlanArrays(n, np.array([1 if k == "emb" else 0 for k in kinds], np.int8), None, 1, 1) for _ in models]
rb = [dp.plan_resident_bytes(mm, p) for mm, p in zip(models, plans)]
print("rb", rb[:2], "arena", len(base.arena()))
budget = int(3.5 * rb[0])
arr, inst = synth.make_poisson_trace(60, 1000.0, 8, seed=5)
res = dp.serve_run(arr, inst, ngpu=1, per_gpu_budget_bytes=budget, cold_ns=[1], warm_ns=[1], resident_bytes=[1],
                   model_of_instance=np.zeros(8, np.int32), dry_run=False, ctx=c, models=models, plans=plans, batch=1, seq=32)
for r in range(60):
    print(r, inst[r], arr[r], res["decide_ns"][r], res["start_ns"][r], res["finish_ns"][r], res["cold"][r], res["nevicted"][r])
print("resident", [mm.is_resident(0) for mm in models], c.pool_stats(0))
