"""Collect tools/ab_eval.sh warm-forward lines into one JSONL (one line per arm x pass x model,
with the arm's label) for profiles/.  python tools/ab_collect.py OUTDIR label=desc ... > FILE"""
import glob
import json
import os
import sys

o = sys.argv[1]
desc = dict(a.split("=", 1) for a in sys.argv[2:])
for f in sorted(glob.glob(os.path.join(o, "warm_*_*.jsonl"))):
    arm, pas = os.path.basename(f)[5:-6].rsplit("_", 1)
    for line in open(f):
        try:
            d = json.loads(line)
        except ValueError:
            continue
        print(json.dumps({"arm": arm, "arm_desc": desc.get(arm, ""), "pass": int(pas), **d}))
