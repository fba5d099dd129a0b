#!/bin/bash
# SURVEY §8(d) C5 on one GPU: the 4:4:1 BERT-Base / RoBERTa-Base / GPT-2 mix, instance
# count 100..300, Poisson arrivals.  Rate and SLO scaled from the paper's 100 rps /
# 100 ms by (paper PipeSwitch BERT-Base cold 40.51 ms / ours ~4.0 ms) x (1 GPU / 4 GPUs):
# ~250 rps, 10 ms.  Budget: 12.5 all-loaded BERT-Base per GPU (the paper's 100-instance knee on
# 8 GPUs, G23).  usage: bash tools/serve_sweep.sh <out.jsonl>
out=${1:-gpurun_out/serve_sweep.jsonl}
: > $out
for m in 100 140 180 220 260 300; do
  timeout 300 python tools/serve_bench.py --mix bert_base:128:4,roberta_base:384:4,gpt2:1024:1 --instances $m \
    --fit 12.5 --rate 250 --requests 1000 --slo-ms 10 --modes PIPESWITCH,DHA,DHA_LINK >> $out 2>> ${out%.jsonl}.err
done
