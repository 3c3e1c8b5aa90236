#!/bin/bash
# tests, then A/B of the grouping scatter (default build vs build/var/notma) on the C5 bench step
mkdir -p gpurun_out
timeout 420 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "multi or group or dist or C5 or c5 or host" > gpurun_out/t_tma.log 2>&1
echo "tests exit $?" >> gpurun_out/t_tma.log
for i in 1 2; do
  timeout 200 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-latency > gpurun_out/b_tma_$i.json 2>/dev/null
  LAKE_LINNOS_LIB=build/var/notma/liblake_linnos.so timeout 200 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-latency > gpurun_out/b_notma_$i.json 2>/dev/null
done
timeout 120 python scripts/c4_quick.py f16 0,2 > gpurun_out/c4_tma.jsonl 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:group_scatter -c 2 --csv python bench.py --steps 1 --warmup 0 --no-cpu --no-e2e --no-latency > gpurun_out/ncu_scatter_tma.csv 2>/dev/null
