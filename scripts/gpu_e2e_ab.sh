#!/bin/bash
# e2e (host-buffer) A/B of variants: the default bench line's e2e value per build
mkdir -p gpurun_out
for v in "$@"; do
  lib=paper_conf_asplos_finglertyshar23_b200/liblake_linnos.so
  [ "$v" != "base" ] && lib=build/var/$v/liblake_linnos.so
  LAKE_LINNOS_LIB=$lib timeout 200 python bench.py --steps 10 --warmup 3 --no-cpu --no-latency \
    > gpurun_out/e2e_$v.json 2> gpurun_out/e2e_$v.err
  python -c "import json;d=json.loads(open('gpurun_out/e2e_$v.json').read().splitlines()[0]);print('$v', d['e2e']['value']/1e9, d['e2e']['ms_per_step'], d['ms_per_step'])" >> gpurun_out/e2e_summary.txt 2>&1
done
