#!/bin/bash
# Per-CTA GEMM phase traces (instrumented build), then the normal build again.
out=${1:-gpurun_out/gemm_trace.jsonl}
: > $out
DP_NVCC_EXTRA=-DDP_GEMM_TRACE python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
cfgs=${GEMM_TRACE_CFGS:-"128,768,768,32,1 128,768,768,32,4 128,768,3072,32,1 128,768,3072,32,4 128,3072,768,32,1 128,2304,768,32,1 1024,4096,1024,256,1 1024,4096,1024,-256,0 384,4096,1024,128,1 384,4096,1024,-128,0"}
for cfg in $cfgs; do
  IFS=, read M N K BN SP <<< "$cfg"
  timeout 60 python tools/gemm_trace.py $M $N $K 20 $BN $SP >> $out 2>&1
done
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
