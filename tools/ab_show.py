"""Summarise tools/ab_eval.sh output: warm-forward medians per arm and pass, GEMM kbench per arm."""
import glob
import json
import os
import sys

o = sys.argv[1]
rows = {}
for f in sorted(glob.glob(os.path.join(o, "warm_*_*.jsonl"))):
    arm, pas = os.path.basename(f)[5:-6].rsplit("_", 1)
    for line in open(f):
        try:
            d = json.loads(line)
        except ValueError:
            continue
        rows.setdefault(f"{d['model']}:{d['seq']}", {}).setdefault(arm, []).append(d["warm_ms_median"])
for k, v in rows.items():
    print(k, "  ".join(f"{a}={'/'.join(str(x) for x in t)}" for a, t in v.items()))
kb = {os.path.basename(f)[len("kbench_gemm_"):-5]: json.load(open(f)) for f in glob.glob(os.path.join(o, "kbench_gemm_*.json"))
      if os.path.getsize(f) > 0}
if kb:
    arms = list(kb)
    print("gemm", arms)
    for k in kb[arms[0]]:
        if k.startswith("gemm_tc"):
            print(k, [kb[a].get(k, {}).get("us") for a in arms])
