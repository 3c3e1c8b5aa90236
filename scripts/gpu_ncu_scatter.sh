mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:group_scatter -s 1 -c 1 \
    -o gpurun_out/prof_scatter python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-latency > gpurun_out/prof_scatter.out 2>&1
