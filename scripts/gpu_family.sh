#!/bin/bash
# NEXT-4: family parity tests, then the family bench (latency sweep + 2^24-row throughput)
mkdir -p gpurun_out
T=${1:-x}
timeout 600 python -m pytest tests/test_gpu_family.py -q -x -rf -p no:cacheprovider > gpurun_out/tfam_$T.log 2>&1
echo "tests exit $?" >> gpurun_out/tfam_$T.log
timeout 900 python bench.py --mode family --sweep-out gpurun_out/family_$T.jsonl > gpurun_out/family_$T.out 2> gpurun_out/family_$T.err
echo "bench exit $?" >> gpurun_out/family_$T.err
