#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "fp32 or server or auto or graph" -p no:cacheprovider > gpurun_out/t_fp32.log 2>&1
echo "exit $?" >> gpurun_out/t_fp32.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_lat.json 2> gpurun_out/bench_lat.err
