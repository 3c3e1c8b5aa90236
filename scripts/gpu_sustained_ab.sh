#!/bin/bash
# sustained (power-capped) A/B: c5_sustained.py STEPS per build, 15 s idle between runs
mkdir -p gpurun_out
STEPS=${STEPS:-400}
for v in "$@"; do
  lib=paper_conf_asplos_finglertyshar23_b200/liblake_linnos.so
  [ "$v" != "base" ] && lib=build/var/$v/liblake_linnos.so
  sleep 15
  echo "== $v" >> gpurun_out/sustained_ab.txt
  LAKE_LINNOS_LIB=$lib timeout 300 python scripts/c5_sustained.py $STEPS > gpurun_out/sus_$v.txt 2>&1
  python - "$v" >> gpurun_out/sustained_ab.txt <<'PY'
import json, sys
v = sys.argv[1]
L = [json.loads(l) for l in open(f"gpurun_out/sus_{v}.txt") if l.startswith("{")]
blk = [l["ms_mean"] for l in L if "steps" in l]
smp = [l for l in L if "t_ms" in l]
late = smp[len(smp) // 2:]
print(json.dumps(dict(variant=v, first_block_ms=blk[0], late_ms=round(sum(blk[len(blk)//2:]) / len(blk[len(blk)//2:]), 4),
                      late_sm_mhz=round(sum(s["sm_mhz"] for s in late) / max(len(late), 1)),
                      late_power_w=round(sum(s["power_w"] for s in late) / max(len(late), 1)))))
PY
done
