#!/bin/bash
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
    --log-file gpurun_out/launches_c5.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/launches_c5.out 2>&1
echo "ncu1 exit $?" >> gpurun_out/launches_c5.out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc_kernel -s 1 -c 1 \
    -o gpurun_out/prof_tc_c5 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/prof_tc_c5.out 2>&1
echo "ncu2 exit $?" >> gpurun_out/prof_tc_c5.out
