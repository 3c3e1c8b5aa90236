#!/bin/bash
# one optimisation iteration: TC tests, bench, trace (no ncu)
mkdir -p gpurun_out
TAG=${1:-x}
timeout 300 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "tc or multi or c3" > gpurun_out/t_$TAG.log 2>&1
echo "tests exit $?" >> gpurun_out/t_$TAG.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
echo "bench exit $?" >> gpurun_out/bench_$TAG.err
LAKE_LINNOS_LIB=build/trace/liblake_linnos_trace.so timeout 300 python scripts/trace_tc.py C5 f16 > gpurun_out/trace_$TAG.txt 2>&1
