#!/bin/bash
# Round-2 profiling evidence (one gpurun call): ncu launch list of the default bench, ncu --set
# full of the kernels changed or added in round 2 (tcgen05 GEMM with the TMA-store epilogue,
# tcgen05 attention K5t, the DHA LayerNorm / embedding cluster broadcast, the fp32 kernels), kbench.
tag=${1:-r02}
o=gpurun_out/$tag
mkdir -p $o
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
export DP_BENCH_UNDER_NCU=1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $o/ncu_bench_launches.csv \
  python bench.py --steps 3 --warmup 3 --profile-iters 1 --no-cpu-baseline --quick > $o/ncu_bench.log 2>&1
unset DP_BENCH_UNDER_NCU
full() {  # name kbench-arg kernel-regex skip
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:"$3" -s $4 -c 1 \
    -o $o/full_$1 -f python tools/kbench.py $2 3 > $o/full_$1.log 2>&1
  ncu -i $o/full_$1.ncu-rep --page raw --csv > $o/full_$1.raw.csv 2>/dev/null
  ncu -i $o/full_$1.ncu-rep --page details --csv > $o/full_$1.details.csv 2>/dev/null
  [ $(stat -c %s $o/full_$1.ncu-rep 2>/dev/null || echo 0) -gt 6000000 ] && rm -f $o/full_$1.ncu-rep
}
full gemm_q gemm gemm_tc 3
full gemm_fc1 gemm gemm_tc 9
full gemm_M384_N4096_K1024 gemm gemm_tc 27
full gemm_M1024_N4096_K1024 gemm gemm_tc 45
full attention_s128 attn attention 3
full attention_s384 attn attention 9
full attention_s1024_causal attn attention 15
full embed_dha embed embed 3
full layernorm_dha lnhost layernorm 3
full skinny_dha skinny skinny 3
full fp32_linear_dha fp32 linear_f32 3
python tools/kbench.py all 50 > $o/kbench.json 2>&1
echo evidence-done
