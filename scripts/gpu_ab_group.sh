#!/bin/bash
# A/B grouping variants: multi-model parity tests, then the default C5 bench step (group +
# fused kernel) and the ncu launch list of the group kernels
mkdir -p gpurun_out
out=gpurun_out/abg_${1:-x}.txt
: > $out
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  echo "$(basename $v) | $(timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nn_pipe.py -m gpu -q -x -p no:cacheprovider -k 'multi or host or c5' 2>&1 | tail -1)" >> $out
done
for rep in 1 2; do
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  b=$(timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(f\"{d['value']/1e9:.4f} Ginf/s step {d['ms_per_step']} ms kernel {r['kernel_ms']:.3f} ms\")")
  echo "$(basename $v) | C5 | $b" >> $out
done
done
for v in build/var/*/; do
  export LAKE_LINNOS_LIB=$v/liblake_linnos.so
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:group -c 40 --csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e 2>/dev/null | grep -E 'group_(hist|scatter)' | awk -F'","' -v n=$(basename $v) '{print n, $5, $NF}' | tail -4 >> $out
done
