#!/bin/bash
# bounded: tests (TC subset), bench C5, one ncu --set full capture of the fused TC kernel
mkdir -p gpurun_out
TAG=${1:-x}
timeout 300 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "tc or multi or c3" > gpurun_out/t_$TAG.log 2>&1
echo "tests exit $?" >> gpurun_out/t_$TAG.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
echo "bench exit $?" >> gpurun_out/bench_$TAG.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc_kernel -s 1 -c 1 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/prof_$TAG.out 2>&1
echo "ncu exit $?" >> gpurun_out/prof_$TAG.out
