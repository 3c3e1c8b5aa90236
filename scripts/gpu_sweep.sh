#!/bin/bash
mkdir -p gpurun_out
T=${1:-x}
timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/tgpu_$T.log 2>&1; echo "tests exit $?" >> gpurun_out/tgpu_$T.log
timeout 900 python bench.py --mode sweep --sweep-out gpurun_out/sweep_$T.jsonl > gpurun_out/sweep_$T.out 2> gpurun_out/sweep_$T.err
