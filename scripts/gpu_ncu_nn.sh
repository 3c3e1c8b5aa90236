#!/bin/bash
mkdir -p gpurun_out
python scripts/run_single.py C3 f16 0 20 > gpurun_out/nn_single.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mlp_tc -s 2 -c 1 \
    -o gpurun_out/prof_nn python scripts/run_single.py C3 f16 0 1 > gpurun_out/prof_nn.out 2>&1
