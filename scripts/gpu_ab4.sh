#!/bin/bash
# A/B: NN-pipeline tests + parity subset once per variant, then C5 and C4 per arch, twice
mkdir -p gpurun_out
out=gpurun_out/ab_${1:-x}.txt
: > $out
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  echo "$(basename $v) | $(timeout 300 python -m pytest tests/test_gpu_nn_pipe.py tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider 2>&1 | tail -1)" >> $out
done
for rep in 1 2; do
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  for cfg in "C5" "C4 --arch 0" "C4 --arch 2" "C3 --arch 0"; do
    b=$(timeout 200 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(f\"{d['value']/1e9:.3f} Ginf/s kernel {r['kernel_ms']:.3f} ms frac {r['frac']:.4f}\")")
    echo "$(basename $v) | $cfg | $b" >> $out
  done
done
done
