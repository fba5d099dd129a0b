#!/bin/bash
# Round-2 (second session) profiling evidence, one gpurun call: the default bench's ncu launch
# list (kernel shares of a BERT-Base k = 1 cold-start step) and ncu --set full of the kernels
# changed this session (tcgen05 GEMM with multi-chunk 3D TMA stages and compile-time epilogues,
# K5t variants), plus the device times of every kernel.
tag=${1:-r02s2}
o=gpurun_out/$tag
mkdir -p $o
export DP_BENCH_UNDER_NCU=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $o/ncu_bench_launches.csv \
  python bench.py --steps 3 --warmup 3 --profile-iters 1 --no-cpu-baseline --quick > $o/ncu_bench.log 2>&1
unset DP_BENCH_UNDER_NCU
full() {  # name kbench-arg kernel-regex skip
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:"$3" -s $4 -c 1 \
    -o $o/full_$1 -f python tools/kbench.py $2 3 > $o/full_$1.log 2>&1
  ncu -i $o/full_$1.ncu-rep --page details --csv > $o/full_$1.details.csv 2>/dev/null
  ncu -i $o/full_$1.ncu-rep --page raw --csv > $o/full_$1.raw.csv 2>/dev/null
  rm -f $o/full_$1.ncu-rep
}
full gemm_q gemm gemm_tc 3
full gemm_fc1 gemm gemm_tc 9
full gemm_fc2 gemm gemm_tc 15
full gemm_M384_N1024_K1024 gemm gemm_tc 21
full gemm_M384_N4096_K1024 gemm gemm_tc 27
full gemm_M1024_N4096_K1024 gemm gemm_tc 45
full gemm_M1024_N1024_K4096 gemm gemm_tc 51
full attention_tc_s384 attn_tc attention_tc 9
full attention_tc_s1024_causal attn_tc attention_tc 15
python tools/kbench.py all 50 > $o/kbench.json 2>&1
echo evidence-done
