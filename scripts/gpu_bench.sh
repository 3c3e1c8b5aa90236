#!/bin/bash
# One GPU session: bench (default C5), ncu launch list, ncu full capture of the fused kernel.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt 2>&1
lscpu | grep -E "Model name|^CPU\(s\)" > gpurun_out/lscpu.txt
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
echo "bench exit $?" >> gpurun_out/bench_c5.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_c5.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/launches_c5.out 2>&1
echo "ncu1 exit $?" >> gpurun_out/launches_c5.out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mlp_tc_kernel -s 1 -c 1 \
    -o gpurun_out/prof_tc_c5 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/prof_tc_c5.out 2>&1
echo "ncu2 exit $?" >> gpurun_out/prof_tc_c5.out
timeout 900 python bench.py --mode sweep --sweep-out gpurun_out/sweep.jsonl > gpurun_out/sweep.out 2> gpurun_out/sweep.err
echo "sweep exit $?" >> gpurun_out/sweep.err
