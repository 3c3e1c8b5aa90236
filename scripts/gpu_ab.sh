#!/bin/bash
# A/B timing of library variants (make variant VAR=name DEFS=...): C5 bench per variant
# usage: bash scripts/gpu_ab.sh var1 var2 ...   ("base" = the product build)
mkdir -p gpurun_out
for v in "$@"; do
  lib=paper_conf_asplos_finglertyshar23_b200/liblake_linnos.so
  [ "$v" != "base" ] && lib=build/var/$v/liblake_linnos.so
  LAKE_LINNOS_LIB=$lib timeout 120 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-latency \
    > gpurun_out/ab_$v.json 2> gpurun_out/ab_$v.err
  python -c "import json;d=json.loads(open('gpurun_out/ab_$v.json').read().splitlines()[0]);print('$v', d['roofline']['kernel_ms'], d['ms_per_step'])" >> gpurun_out/ab_summary.txt 2>&1
done
