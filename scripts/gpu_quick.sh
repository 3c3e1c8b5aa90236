#!/bin/bash
# tests (bounded) then a bounded bench run
mkdir -p gpurun_out
timeout 420 python -m pytest tests -m gpu -q -rf -x -p no:cacheprovider > gpurun_out/t_all.log 2>&1
echo "tests exit $?" >> gpurun_out/t_all.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
echo "bench exit $?" >> gpurun_out/bench_c5.err
