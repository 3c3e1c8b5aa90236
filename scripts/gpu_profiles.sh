#!/bin/bash
# Evidence for profiles/: ncu launch list of the default bench command and one ncu --set full
# capture of the dominant kernel (fused tcgen05 MLP), plus the digitise kernel at C5 size.
mkdir -p gpurun_out
TAG=${1:-r1}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu \
    > gpurun_out/launches_$TAG.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc_kernel -s 3 -c 1 \
    -o gpurun_out/full_tc_$TAG python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu \
    > gpurun_out/full_tc_$TAG.out 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_fp32_kernel -s 1 -c 1 \
    -o gpurun_out/full_fp32_$TAG python bench.py --config C3 --prec fp32 --steps 1 --warmup 1 --no-e2e --no-cpu \
    > gpurun_out/full_fp32_$TAG.out 2>&1
timeout 300 ncu --set full --clock-control none -k regex:digitize_kernel -c 1 \
    -o gpurun_out/full_dig_$TAG python scripts/run_digitize.py > gpurun_out/full_dig_$TAG.out 2>&1
for m in mllb kml; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:mlp_family -s 1 -c 1 \
      -o gpurun_out/full_fam${m}_$TAG python scripts/run_family.py $m > gpurun_out/full_fam${m}_$TAG.out 2>&1
done
echo done
