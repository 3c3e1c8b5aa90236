"""Per-source-line warp-stall samples from an ncu report (needs -lineinfo).
usage: python scripts/ncu_lines.py report.ncu-rep [n]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
cur_file, hdr, out = None, None, []
for r in rows:
    if r and r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 5 or r[0] == "":
        continue
    d = dict(zip(hdr, r))
    try:
        s = int(r[4] or 0)
    except ValueError:
        continue
    stalls = {k[6:]: int(v) for k, v in d.items() if k.startswith("stall_") and "Not Issued" not in k and v.isdigit() and int(v) > 0}
    top = sorted(stalls.items(), key=lambda x: -x[1])[:3]
    out.append((s, f"{cur_file}:{r[0]}", r[1][:60], top))
tot = sum(x[0] for x in out)
for s, loc, src, top in sorted(out, key=lambda x: -x[0])[:n]:
    print(f"{100 * s / tot:5.1f}% {loc:22s} {src:60s} {top}")
