#!/bin/bash
# compute-sanitizer over sanitize_run.py (every kernel, small sizes), then the grouping kernels
# alone on a multi-chunk-per-block size (LAKE_SAN_BIG)
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_run.py > gpurun_out/san_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/san_$tool.txt
done
for tool in memcheck racecheck synccheck; do
  LAKE_SAN_BIG=1 timeout 900 compute-sanitizer --tool $tool --print-limit 20 --kernel-regex kns=group \
      python scripts/sanitize_run.py > gpurun_out/san_big_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/san_big_$tool.txt
done
