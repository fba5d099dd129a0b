DP_NVCC_EXTRA=-DDP_INSTRUMENT python paper_conf_eurosys_jeongba23_b200/build.py > gpurun_out/build.log 2>&1
DP_GEMM_BN=96 timeout 300 python -m pytest -q tests/test_gpu_kernels.py -k "gemm or linear" > gpurun_out/pytest_bn96.log 2>&1
for bn in 0 64 96 128; do echo "== BN=$bn" >> gpurun_out/bn_sweep.txt; DP_GEMM_BN=$bn DP_GEMM_SPLIT=1 python tools/kbench.py gemm 30 2>&1 | python -c "
import json,sys
d=json.load(sys.stdin)
for k,v in d.items():
    if k.startswith('gemm'): print(k, v['us'], v.get('tflops'))
" >> gpurun_out/bn_sweep.txt; done
echo "== model" >> gpurun_out/bn_sweep.txt
python tools/kbench.py gemm 30 >> gpurun_out/bn_sweep.txt 2>&1
python paper_conf_eurosys_jeongba23_b200/build.py > /dev/null 2>&1
tail -1 gpurun_out/pytest_bn96.log
