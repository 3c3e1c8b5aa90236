#!/bin/bash
# Rehearsal of the driver's round-end sequence on one GPU.
mkdir -p gpurun_out
T=${1:-x}
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$T.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke_$T.log
timeout 600 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/tgpu_$T.log 2>&1; echo "tests exit $?" >> gpurun_out/tgpu_$T.log
timeout 600 python bench.py > gpurun_out/bench_full_$T.json 2> gpurun_out/bench_full_$T.err; echo "bench exit $?" >> gpurun_out/bench_full_$T.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$T.json 2> gpurun_out/bench_ref_$T.err
timeout 900 python bench.py --mode sweep --sweep-out gpurun_out/sweep_$T.jsonl > gpurun_out/sweep_$T.out 2> gpurun_out/sweep_$T.err
