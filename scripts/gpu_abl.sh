#!/bin/bash
# timing-only A/B of the variants under build/var/* (no parity: ablations break numerics)
mkdir -p gpurun_out
out=gpurun_out/abl_${1:-x}.txt
: > $out
for v in build/var/*/; do
  name=$(basename $v)
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  b=$(timeout 200 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(f\"kernel {r['kernel_ms']:.3f} ms frac {r['frac']:.4f}\")")
  echo "$name | $b" >> $out
done
