#!/bin/bash
# GPU session: correctness of the split-K GEMM + cluster skinny kernel, then timings / traces.
o=gpurun_out/${1:-g2}
mkdir -p $o
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
timeout 600 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -15 > $o/tests.log
timeout 120 python tools/kbench.py skinny > $o/kb_skinny.json 2>&1
timeout 120 python tools/kbench.py all > $o/kb_all.json 2>&1
bash tools/gemm_sweep.sh $o/sweep.txt "${2:-1 2 4 6 8}" > /dev/null 2>&1
DP_NVCC_EXTRA=-DDP_GEMM_TRACE python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
for shape in "128 768 768" "128 768 3072" "128 3072 768"; do
  for sp in 1 2 4 6; do
    DP_GEMM_BN=32 DP_GEMM_SPLIT=$sp timeout 60 python tools/gemm_trace.py $shape >> $o/trace.jsonl 2>&1
  done
done
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
timeout 300 python bench.py --no-cpu-baseline > $o/bench.json 2> $o/bench.err
echo g2-done
