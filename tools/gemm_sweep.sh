#!/bin/bash
# GEMM tile/split sweep on the GPU box: python tools/kbench.py gemm under DP_GEMM_BN/SPLIT overrides.
out=${1:-gpurun_out/gemm_sweep.txt}
splits=${2:-"1 2 4"}
: > "$out"
for bn in 32 64 128 256; do
  for sp in $splits; do
    echo "== BN=$bn SPLIT=$sp" >> "$out"
    DP_GEMM_BN=$bn DP_GEMM_SPLIT=$sp timeout 120 python tools/kbench.py gemm 30 2>&1 | python -c "
import json,sys
d=json.load(sys.stdin)
for k,v in d.items():
    if k.startswith('gemm'): print(k, v['us'])
" >> "$out" 2>&1
  done
done
