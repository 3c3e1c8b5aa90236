#!/bin/bash
# FP32-path checks: bit-exact parity subset + C3 NN+2 / NN+1 FP32 timing (run_single)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "fp32 or server or auto or graph or c3 or c5" -p no:cacheprovider > gpurun_out/t_fp32.log 2>&1
echo "exit $?" >> gpurun_out/t_fp32.log
for a in 2 1 0; do python scripts/run_single.py C3 fp32 $a 5; done > gpurun_out/fp32_single.txt 2>&1
