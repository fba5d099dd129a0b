timeout 300 python -m pytest -q tests/test_gpu_kernels.py -k "attention_tc" > gpurun_out/pytest_attn5.log 2>&1; tail -1 gpurun_out/pytest_attn5.log
timeout 120 python tools/kbench.py attn 50 > gpurun_out/kbench_attn5.json 2>&1
DP_NVCC_EXTRA=-DDP_ATT_TRACE python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null 2>&1; rm -f gpurun_out/att_trace.jsonl
for c in "1024 1024 16 1" "384 1024 16 0" "128 768 12 0"; do timeout 60 python tools/att_trace.py $c >> gpurun_out/att_trace.jsonl 2>&1; done
