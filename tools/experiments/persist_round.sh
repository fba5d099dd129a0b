#!/bin/bash
# K6 iteration on the GPU box: parity tests, warm bench, then the per-op trace (instrumented
# build), then the normal build again.  Outputs under gpurun_out/.
mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_persist.py -x -q > gpurun_out/persist.log 2>&1; echo rc=$? >> gpurun_out/persist.log
timeout 300 python tools/warm_bench.py ${WARM_SPECS:-bert_base:128 gpt2:256} > gpurun_out/warm.log 2>&1
DP_NVCC_EXTRA=-DDP_PERSIST_TRACE python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
DP_PERSIST_VERBOSE=1 timeout 120 python tools/persist_trace.py ${TRACE_SPEC:-bert_base 128} > gpurun_out/ptrace.log 2>&1; echo rc=$? >> gpurun_out/ptrace.log
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null
