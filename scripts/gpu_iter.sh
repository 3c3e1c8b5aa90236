mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -p no:cacheprovider -k "tc_tolerance or digits_equals_raw or bf16 or batch_indep" > gpurun_out/t_tc.log 2>&1
echo "exit $?" >> gpurun_out/t_tc.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_f16.json 2> gpurun_out/bench_f16.err
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --prec tf32 > gpurun_out/bench_tf32.json 2> gpurun_out/bench_tf32.err
timeout 900 python bench.py --mode report > gpurun_out/report.out 2> gpurun_out/report.err
