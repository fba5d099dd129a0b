#!/bin/bash
# the 4:4:1 BERT-Base / RoBERTa-Base / GPT-2 mix, instance count
# 100..300, Poisson arrivals, served live by the online dispatcher (R11-live) on G GPUs.
# Rate and SLO scaled from the paper's 100 rps / 100 ms by (paper PipeSwitch BERT-Base cold
# 40.51 ms / ours ~4.0 ms) x (G GPUs / 4 GPUs): ~250 rps per GPU, 10 ms.  Budget: 12.5 all-loaded
# BERT-Base per GPU (the paper's 100-instance knee on 8 GPUs, G23).  With G > 1 the PT_DHA_LINK
# mode borrows idle GPUs' links for cold starts.
# usage: bash tools/serve_sweep.sh <out.jsonl> [G]
out=${1:-gpurun_out/serve_sweep.jsonl}
G=${2:-1}
modes="PIPESWITCH,DHA,DHA_LINK"
[ "$G" -gt 1 ] && modes="$modes,PT_DHA_LINK"
: > $out
for m in 100 140 180 220 260 300; do
  timeout 600 python tools/serve_bench.py --gpus $G --mix bert_base:128:4,roberta_base:384:4,gpt2:1024:1 \
    --instances $m --fit 12.5 --rate $((250 * G)) --requests 1000 --slo-ms 10 --modes $modes >> $out 2>> ${out%.jsonl}.err
done
