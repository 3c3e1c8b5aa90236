#!/bin/bash
# End-of-session evidence: ncu profile set, full default bench + reference arm, C2 sweep.
TAG=${1:-r1c}
mkdir -p gpurun_out
bash scripts/gpu_profiles.sh $TAG
timeout 600 python bench.py > gpurun_out/bench_full_$TAG.json 2> gpurun_out/bench_full_$TAG.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
