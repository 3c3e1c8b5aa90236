#!/bin/bash
# ncu launch list (per-launch durations, cold caches) of the default C5 bench command
TAG=${1:-x}; shift
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu --no-latency "$@" \
    > gpurun_out/launches_$TAG.out 2>&1
echo "exit $?" >> gpurun_out/launches_$TAG.out
