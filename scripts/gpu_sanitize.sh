#!/bin/bash
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_run.py > gpurun_out/san_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/san_$tool.txt
done
