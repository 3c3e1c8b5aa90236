#!/bin/bash
# A/B of the NN output-layer split (LAKE_OTC_KSTEPS variants under build/var/otcK) + default
mkdir -p gpurun_out
for v in "$@"; do
  echo "== $v" >> gpurun_out/otc_ab.jsonl
  if [ "$v" = default ]; then
    timeout 120 python scripts/c4_quick.py f16 0 >> gpurun_out/otc_ab.jsonl 2>&1
  else
    LAKE_LINNOS_LIB=build/var/$v/liblake_linnos.so timeout 120 python scripts/c4_quick.py f16 0 >> gpurun_out/otc_ab.jsonl 2>&1
  fi
done
