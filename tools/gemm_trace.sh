#!/bin/bash
# Per-CTA GEMM phase traces (instrumented build), then the normal build again.
out=${1:-gpurun_out/gemm_trace.jsonl}
: > $out
DP_NVCC_EXTRA=-DDP_GEMM_TRACE python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
for cfg in "128 768 768 32 1" "128 768 768 32 4" "128 768 3072 32 1" "128 768 3072 32 4" "128 3072 768 32 1" "128 2304 768 32 1" "1024 4096 1024 256 1"; do
  set -- $cfg
  DP_GEMM_BN=$4 DP_GEMM_SPLIT=$5 timeout 60 python tools/gemm_trace.py $1 $2 $3 >> $out 2>&1
done
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
