#!/bin/bash
# round profiles: full GPU suite, smoke, default bench line, ncu launch list + full capture of
# the fused kernel (C5), report mode
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/t_all.log 2>&1
echo "exit $?" >> gpurun_out/t_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
echo "exit $?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/launches_r2.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/launches_r2.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc -s 1 -c 1 \
    -o gpurun_out/prof_r2_tc python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/prof_r2_tc.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:group_scatter -s 1 -c 1 \
    -o gpurun_out/prof_r2_scatter python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/prof_r2_scatter.out 2>&1
