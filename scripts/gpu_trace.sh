#!/bin/bash
# timeline traces of the tcgen05 kernel: SMEM-log trace build (make variant VAR=tsmem
# DEFS="-DLAKE_TRACE -DLAKE_TRACE_SMEM"); args: config prec [arch]
mkdir -p gpurun_out
LAKE_TRACE_CAP=512 LAKE_LINNOS_LIB=build/var/tsmem/liblake_linnos.so timeout 300 python scripts/trace_tc.py "$@" > gpurun_out/trace_smem_$1_$3.txt 2>&1
echo "exit $?" >> gpurun_out/trace_smem_$1_$3.txt
