mkdir -p gpurun_out/ab
export DP_PT_CASES=PIPESWITCH/1,PT_DHA_LINK_BAL/8,PT_DHA_LINK_STRIPE/8,PT_DHA_LINK_STRIPE/4
timeout 600 python tools/pt_transport_bench.py bert_base 128 10 > gpurun_out/ab/coalesce.jsonl 2>&1
DP_NO_WAIT_COALESCE=1 timeout 600 python tools/pt_transport_bench.py bert_base 128 10 > gpurun_out/ab/nocoalesce.jsonl 2>&1
timeout 900 python -m pytest tests/test_gpu_pt_forward.py tests/test_gpu_forward.py -x -q > gpurun_out/ab/tests.log 2>&1; echo rc=$? >> gpurun_out/ab/tests.log
