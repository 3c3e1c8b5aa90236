#!/bin/bash
# iteration script: tensor-core parity subset + C5 bench + C4 report
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nn_pipe.py -m gpu -q -rf -x -p no:cacheprovider -k "tc_ or digits_equals_raw or bf16 or batch_indep or multi or c3 or c5 or single_model or narrow or host" > gpurun_out/t_tc.log 2>&1
echo "exit $?" >> gpurun_out/t_tc.log
timeout 120 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-latency > gpurun_out/bench_f16.json 2> gpurun_out/bench_f16.err
echo "exit $?" >> gpurun_out/bench_f16.err
timeout 600 python bench.py --mode report > gpurun_out/report.out 2> gpurun_out/report.err
python scripts/run_single.py C3 f16 0 20 > gpurun_out/nn_single.txt 2>&1
python scripts/run_single.py C3 f16 2 20 >> gpurun_out/nn_single.txt 2>&1
