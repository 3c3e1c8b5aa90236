#!/bin/bash
# ncu launch list + one full capture of each tensor-core kernel on the C5 bench command
# usage: bash scripts/gpu_ncu.sh TAG [extra bench args]
TAG=${1:-x}; shift
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu "$@" \
    > gpurun_out/launches_$TAG.out 2>&1
echo "ncu1 exit $?" >> gpurun_out/launches_$TAG.out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc -s 1 -c 1 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" \
    > gpurun_out/prof_$TAG.out 2>&1
echo "ncu2 exit $?" >> gpurun_out/prof_$TAG.out
