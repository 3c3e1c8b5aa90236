mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dist.py -m gpu -q -rf -p no:cacheprovider > gpurun_out/t_dist.log 2>&1
echo "exit $?" >> gpurun_out/t_dist.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
echo "exit $?" >> gpurun_out/bench_full.err
