#!/bin/bash
# r1d closing run: round-end rehearsal + report/family tables + family ncu captures
mkdir -p gpurun_out
T=r1d2
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$T.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke_$T.log
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/tgpu_$T.log 2>&1; echo "tests exit $?" >> gpurun_out/tgpu_$T.log
timeout 600 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref_$T.json 2> gpurun_out/bench_ref_$T.err
timeout 900 python bench.py --mode report --sweep-out gpurun_out/report_$T.jsonl > gpurun_out/report_$T.out 2> gpurun_out/report_$T.err
timeout 900 python bench.py --mode family --sweep-out gpurun_out/family_$T.jsonl > gpurun_out/family_$T.out 2> gpurun_out/family_$T.err
for m in mllb kml; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:mlp_family -s 1 -c 1 \
      -o gpurun_out/full_fam${m}_$T python scripts/run_family.py $m > gpurun_out/full_fam${m}_$T.out 2>&1
done
echo done
