#!/bin/bash
# timeline traces of the tcgen05 kernels (trace build; scripts/trace_tc.py, trace_tc2.py)
mkdir -p gpurun_out
LAKE_LINNOS_LIB=build/trace/liblake_linnos_trace.so timeout 300 python scripts/trace_tc2.py C5 f16 > gpurun_out/trace2_c5.txt 2>&1
echo "exit $?" >> gpurun_out/trace2_c5.txt
