#!/bin/bash
# One gpurun call that gathers the profiling evidence kept under profiles/:
#   ncu launch list of the bench command, ncu --set full of each hot kernel (via kbench),
#   planner comparison on real profiles, and the serving benchmark with the paper's model mix.
# usage (on the GPU box): bash tools/evidence.sh <tag>
tag=${1:-r01}
o=gpurun_out/$tag
mkdir -p $o
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
export DP_BENCH_UNDER_NCU=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $o/ncu_bench_launches.csv \
  python bench.py --steps 3 --warmup 3 --profile-iters 1 --no-cpu-baseline > $o/ncu_bench.log 2>&1
unset DP_BENCH_UNDER_NCU
full() {  # name kbench-arg kernel-regex skip
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:"$3" -s $4 -c 1 \
    -o $o/full_$1 -f python tools/kbench.py $2 3 > $o/full_$1.log 2>&1
  ncu -i $o/full_$1.ncu-rep --page raw --csv > $o/full_$1.raw.csv 2>/dev/null
  ncu -i $o/full_$1.ncu-rep --page details --csv > $o/full_$1.details.csv 2>/dev/null
  # keep the report itself only if small (gpurun merges at most 64 MiB back)
  [ $(stat -c %s $o/full_$1.ncu-rep 2>/dev/null || echo 0) -gt 6000000 ] && rm -f $o/full_$1.ncu-rep
}
full gemm_q gemm gemm_tc 3
full gemm_fc1 gemm gemm_tc 9
full gemm_fc2 gemm gemm_tc 15
full skinny_dha skinny skinny 3
full embed_dha embed embed 3
full attention attn attention 3
full layernorm ln layernorm 3
full lmhead_hbm lmhead gemv 16
full attention_k5b attn attention2 3
full pt_forward ptfwd pt_forward 12
timeout 1500 python tools/plan_compare.py > $o/plan_compare.json 2> $o/plan_compare.err
timeout 600 python tools/dump_costs.py > $o/cost_tables.json 2> $o/cost_tables.err
timeout 300 python tools/torch_warm_baseline.py bert_base:128 bert_large:384 gpt2:256 gpt2_medium:1024 > $o/warm_vs_torch.jsonl 2>&1
python bench.py > $o/bench.log 2>&1
timeout 600 python tools/serve_bench.py --mix bert_base:128:4,roberta_base:384:4,gpt2:1024:1 --instances 45 \
  --fit 8 --rate 200 --requests 600 --slo-ms 20 > $o/serve_mix.json 2> $o/serve_mix.err
echo evidence-done
