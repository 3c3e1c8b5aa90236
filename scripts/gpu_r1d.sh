#!/bin/bash
# r1d evidence run: bench lines (ours + reference arm + family), then the ncu captures
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_r1d.json 2> gpurun_out/bench_r1d.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_r1d.json 2> gpurun_out/bench_ref_r1d.err
timeout 900 python bench.py --mode family --sweep-out gpurun_out/family_r1d.jsonl > gpurun_out/family_r1d.out 2> gpurun_out/family_r1d.err
bash scripts/gpu_profiles.sh r1d
