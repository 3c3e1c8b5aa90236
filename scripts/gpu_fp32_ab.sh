#!/bin/bash
# FP32 A/B: C3 (2^20 I/Os) FP32 timing per arch for the default build and build/var/<v>
# variants, plus the bit-exact FP32 parity subset on each variant
mkdir -p gpurun_out
for v in "$@"; do
  if [ "$v" = default ]; then L=""; else L=build/var/$v/liblake_linnos.so; fi
  echo "== $v" >> gpurun_out/fp32_ab.txt
  for a in 2 1; do
    if [ -n "$L" ]; then LAKE_LINNOS_LIB=$L timeout 120 python scripts/run_single.py C3 fp32 $a 5; else timeout 120 python scripts/run_single.py C3 fp32 $a 5; fi
  done >> gpurun_out/fp32_ab.txt 2>&1
  if [ -n "$L" ]; then
    LAKE_LINNOS_LIB=$L timeout 400 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "fp32 or c3 or c5" -p no:cacheprovider > gpurun_out/t_fp32_$v.log 2>&1
    echo "exit $?" >> gpurun_out/t_fp32_$v.log
  fi
done
