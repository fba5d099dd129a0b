"""Measured output error of full-size cold starts against the fp64 oracle, per storage dtype
("measure and print bf16 max-abs with the fp32 residual stream").

For each model / sequence length / dtype: one cold start (all units loaded, so every linear runs
on the tcgen05 GEMM; plus the default DHA_LINK-style plan with the embeddings by DHA) compared
element by element with the oracle's fp64 forward on the same storage-rounded weights.
Reported per case:
  max_abs        max |gpu - oracle| over last_hidden_state
  max_abs_pool   the same for the pooler output (BERT / RoBERTa)
  floor          max |round_dtype(oracle) - oracle|: the error of an EXACT computation whose
                 result is stored in the output dtype (half an ulp of the largest outputs)
  excess         max_abs - floor (what the kernels' arithmetic adds on top of the output rounding)
  max_rel        max |gpu - oracle| / max(1, |oracle|)
Usage: python tools/precision_report.py [--out FILE] [model:seq ...]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cases", nargs="*", default=["bert_base:128", "bert_large:384", "roberta_large:384",
                                                 "gpt2_medium:1024"])
    ap.add_argument("--dtypes", default="fp16,bf16")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch

    import paper_conf_eurosys_jeongba23_b200 as dp
    from oracle import forward as F

    tdt = {"fp16": torch.float16, "bf16": torch.bfloat16, "fp32": torch.float32}
    ctx = dp.Context([0])
    rows = []
    for case in a.cases:
        name, S = case.split(":")
        S = int(S)
        m = synth.SHAPES[name]
        for dtype in a.dtypes.split(","):
            w = synth.make_weights(m, seed=0, dtype=dtype)
            ids = synth.make_ids(m, 1, S, seed=1)
            ref, ref_pool = F.forward(m, w, ids, dtype)
            ref = ref.reshape(S, -1)
            model = dp.Model(ctx, m, w, dtype)
            n = model.n
            kinds = [u["kind"] for u in model.units()]
            plans = {"all_load": dp._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1),
                     "emb_dha": dp._lib.PlanArrays(n, np.array([1 if k == "emb" else 0 for k in kinds], np.int8),
                                                   None, 3, 1)}
            rounded = synth.storage_to_f64(synth.round_to(ref.astype(np.float32), dtype), dtype)
            floor = float(np.abs(rounded - ref).max())
            for pname, plan in plans.items():
                ids_t = torch.from_numpy(ids).cuda()
                out = torch.empty(S, m.hidden, dtype=tdt[dtype], device="cuda")
                pool = torch.empty(1, m.hidden, dtype=tdt[dtype], device="cuda") if m.family != "gpt2" else None
                model.infer_cold(plan, 0, ids_t, out, pool)
                torch.cuda.synchronize()
                model.evict(0)
                got = out.float().cpu().numpy().astype(np.float64)
                err = np.abs(got - ref)
                row = {"model": name, "seq": S, "dtype": dtype, "plan": pname, "max_abs": float(err.max()),
                       "floor": floor, "excess": float(err.max() - floor),
                       "max_rel": float((err / np.maximum(1.0, np.abs(ref))).max()),
                       "max_abs_ref": float(np.abs(ref).max())}
                # by output magnitude: where 1e-2 is above / below the bf16 output rounding
                for lo, hi in ((0, 1), (1, 2), (2, 4), (4, 1e9)):
                    sel = (np.abs(ref) >= lo) & (np.abs(ref) < hi)
                    row[f"max_abs_ref_{lo}_{hi if hi < 1e9 else 'inf'}"] = float(err[sel].max()) if sel.any() else None
                if pool is not None:
                    row["max_abs_pool"] = float(np.abs(pool.float().cpu().numpy() - ref_pool).max())
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
