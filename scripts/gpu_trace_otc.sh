#!/bin/bash
# timeline of the NN (output-on-tensor-core) kernel: make variant VAR=totc
# DEFS="-DLAKE_TRACE -DLAKE_TRACE_SMEM -DLAKE_TRACE_TW0=30 -DLAKE_TRACE_OTC"; args: config prec arch
# (TVAR=<variant dir> selects another trace build)
mkdir -p gpurun_out
V=${TVAR:-totc}
LAKE_TRACE_OTC=1 LAKE_TRACE_CAP=512 LAKE_LINNOS_LIB=build/var/$V/liblake_linnos.so timeout 300 python scripts/trace_tc.py "$@" > gpurun_out/trace_${V}_$1_$3.txt 2>&1
echo "exit $?" >> gpurun_out/trace_${V}_$1_$3.txt
