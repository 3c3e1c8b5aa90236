#!/bin/bash
# iteration script: quick tensor-core parity + C5 bench A/B (two-tile vs one-tile kernel)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 120 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-latency > gpurun_out/bench_f16.json 2> gpurun_out/bench_f16.err
echo "exit $?" >> gpurun_out/bench_f16.err
LAKE_TC_TWO_TILE=1 timeout 120 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-latency > gpurun_out/bench_f16_2t.json 2> gpurun_out/bench_f16_2t.err
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nn_pipe.py -m gpu -q -rf -x -p no:cacheprovider -k "tc_tolerance or digits_equals_raw or bf16 or batch_indep or multi or c3 or c5 or single_model" > gpurun_out/t_tc.log 2>&1
echo "exit $?" >> gpurun_out/t_tc.log
