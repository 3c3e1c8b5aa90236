#!/bin/bash
# one ncu --set full capture of the fused kernel per library variant (C5 bench command)
# usage: bash scripts/gpu_ncu_ab.sh var1 var2 ...   ("base" = the product build)
mkdir -p gpurun_out
for v in "$@"; do
  lib=paper_conf_asplos_finglertyshar23_b200/liblake_linnos.so
  [ "$v" != "base" ] && lib=build/var/$v/liblake_linnos.so
  LAKE_LINNOS_LIB=$lib timeout 300 ncu --set full --clock-control none --import-source on -k regex:mlp_tc -s 1 -c 1 \
    -o gpurun_out/prof_ab_$v python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-latency \
    > gpurun_out/prof_ab_$v.out 2>&1
done
