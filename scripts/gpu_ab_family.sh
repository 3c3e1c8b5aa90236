#!/bin/bash
# A/B family-kernel variants under build/var/*: family parity tests, then 2^24-row throughput
mkdir -p gpurun_out
out=gpurun_out/abfam_${1:-x}.txt
: > $out
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  echo "$(basename $v) | $(timeout 300 python -m pytest tests/test_gpu_family.py -m gpu -q -x -p no:cacheprovider 2>&1 | tail -1)" >> $out
done
for rep in 1 2; do
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  timeout 300 python scripts/run_family.py --time >> /dev/null 2>&1
  echo "$(basename $v) | $(timeout 300 python scripts/run_family.py --time 2>&1 | tr '\n' ' ')" >> $out
done
done
