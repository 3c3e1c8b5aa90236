#!/bin/bash
# end-of-round measurement pass (r2): full GPU suite, smoke, default bench line, reference
# arm, ncu launch list + full captures (fused C5 kernel, grouping scatter, NN kernel, FP32),
# report mode (C3/C4/C5 + single-model NN), C2 latency sweep
TAG=${1:-r2f}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider --timeout=600 > gpurun_out/t_all.log 2>&1
echo "exit $?" >> gpurun_out/t_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
echo "exit $?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/launches_$TAG.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc -s 1 -c 1 \
    -o gpurun_out/full_tc_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/full_tc_$TAG.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:group_scatter -s 1 -c 1 \
    -o gpurun_out/full_scatter_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/full_scatter_$TAG.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc -s 2 -c 1 \
    -o gpurun_out/full_nn_$TAG python scripts/run_single.py C3 f16 0 1 > gpurun_out/full_nn_$TAG.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_fp32 -s 2 -c 1 \
    -o gpurun_out/full_fp32_$TAG python scripts/run_single.py C3 fp32 2 1 > gpurun_out/full_fp32_$TAG.out 2>&1
timeout 1200 python bench.py --mode report > gpurun_out/report.jsonl 2> gpurun_out/report.err
timeout 900 python bench.py --mode sweep --sweep-out gpurun_out/sweep_c2.jsonl > gpurun_out/sweep.out 2> gpurun_out/sweep.err
