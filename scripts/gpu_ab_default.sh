#!/bin/bash
# default bench command (C5) for each variant under build/var/*, 3 interleaved reps
mkdir -p gpurun_out
out=gpurun_out/abdef_${1:-x}.txt
: > $out
for rep in 1 2 3; do
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  b=$(timeout 300 python bench.py --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(f\"{d['value']/1e9:.3f} Ginf/s step {d['ms_per_step']} kernel {r['kernel_ms']:.3f} ms frac {r['frac']:.4f} clocks {d['clocks']}\")")
  echo "$(basename $v) | $b" >> $out
done
done
