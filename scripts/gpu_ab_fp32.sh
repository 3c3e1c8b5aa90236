#!/bin/bash
# A/B of FP32-path variants under build/var/*: FP32 parity tests, then FP32 throughput
mkdir -p gpurun_out
out=gpurun_out/abf_${1:-x}.txt
: > $out
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  echo "$(basename $v) | $(timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k 'fp32 or FP32 or multi or host or server or c3' 2>&1 | tail -1)" >> $out
done
for rep in 1 2; do
for v in build/var/*/; do
  name=$(basename $v)
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  for cfg in "C3 --prec fp32" "C4 --prec fp32 --arch 2" "C4 --prec fp32 --arch 0"; do
    b=$(timeout 200 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(f\"{d['value']/1e9:.4f} Ginf/s kernel {r['kernel_ms']:.3f} ms {r['achieved']} {r['unit']} frac {r['frac']:.4f}\")")
    echo "$name | $cfg | $b" >> $out
  done
done
done
