"""Mean per-kernel duration / DRAM bytes from an ncu --csv launch list (scripts/gpu_launches.sh)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = None
d = collections.defaultdict(list)
for r in rows:
    if 'Kernel Name' in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        x = dict(zip(hdr, r))
        d[(x['Kernel Name'][:44], x['Metric Name'])].append(float(x['Metric Value'].replace(',', '')))
for k, v in sorted(d.items()):
    print(f"{k[0]:46s} {k[1]:24s} n={len(v):3d} mean={sum(v) / len(v):.6g}")
