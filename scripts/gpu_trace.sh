#!/bin/bash
mkdir -p gpurun_out
LAKE_LINNOS_LIB=build/trace/liblake_linnos_trace.so timeout 300 python scripts/trace_tc.py C5 f16 > gpurun_out/trace_c5.txt 2>&1
echo "exit $?" >> gpurun_out/trace_c5.txt
