#!/bin/bash
# Cold-start latency vs DMA piece size and tail piece (R18): bash tools/tail_sweep.sh <out.jsonl>
out=${1:-gpurun_out/tail_sweep.jsonl}
: > $out
for chunk in 32 64; do
  for tail in 2 6 8 12; do
    timeout 200 python bench.py --quick --no-cpu-baseline --steps 20 --chunk-mb $chunk --tail-mb $tail | \
      python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(json.dumps({'chunk_mb': $chunk, 'tail_mb': $tail, 'ms': d['value'], 'copies': d['stats']['copies'], 'R_alg': d['path_roofline']['R_algorithmic_ms']}))" >> $out
  done
done
# GEMM ring depth vs warm/cold latency (a shallower ring lets the PDL prologue overlap)
for st in 4 6 8; do
  DP_GEMM_STAGES=$st timeout 200 python bench.py --quick --no-cpu-baseline --steps 20 | \
    python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(json.dumps({'gemm_stages': $st, 'ms': d['value'], 'T_warm': d['path_roofline']['T_warm_ms']}))" >> $out
done
