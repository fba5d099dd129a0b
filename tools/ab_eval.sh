#!/bin/bash
# A/B of library builds: warm forwards (tools/warm_bench.py, PDL graph, L2 flushed) and GEMM
# device times (tools/kbench.py gemm), each arm in its own process, all arms run twice in
# alternation.  Arms: AB_ARMS="name:path ..." (path "-" = the in-tree build); default
# "head:ab/lib_head.so new:-"; an arm may add a third field VAR=value (an experiment knob of an
# instrumented build, e.g. DP_GEMM_CFG=128,768,768,32,4).  Usage: tools/ab_eval.sh OUTDIR [specs...]
o=${1:-gpurun_out/ab}; shift
specs=${@:-"bert_base:128 bert_large:384 gpt2_medium:1024"}
arms=${AB_ARMS:-"head:$PWD/ab/lib_head.so new:-"}
mkdir -p $o
for pass in 1 2; do
  for arm in $arms; do
    name=${arm%%:*}; rest=${arm#*:}; path=${rest%%:*}; envs=""
    [ "$rest" != "$path" ] && envs=${rest#*:}   # optional third field: VAR=value (no spaces)
    if [ "$path" = "-" ]; then unset DP_LIB; else export DP_LIB=$path; fi
    env $envs DP_N=50 timeout 600 python tools/warm_bench.py $specs > $o/warm_${name}_$pass.jsonl 2> $o/warm_${name}_$pass.err
    [ $pass = 1 ] && [ -z "$AB_NO_KBENCH" ] && timeout 300 python tools/kbench.py gemm 100 > $o/kbench_gemm_$name.json 2> $o/kbench_gemm_$name.err
    unset DP_LIB
  done
done
