"""Summarise the ncu captures of one round into profiles/ (tracked):
  profiles/<tag>_launches.txt   per-kernel launch list (ncu gpu__time_duration, cold-cache and
                                serialised: compare SHARES of the step, not absolutes)
  profiles/<tag>_<kernel>.txt   headline metrics + top stall sites of each --set full capture
  profiles/traffic.json         dram read+write bytes per launch of the dominant kernel, keyed
                                like bench.py's roofline lookup (<config>_<prec>_g<N>)
usage: python scripts/make_profiles.py <tag> [gpurun_out]"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]
src = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "gpurun_out")
out = os.path.join(ROOT, "profiles")
os.makedirs(out, exist_ok=True)


def raw_metrics(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    return [dict(zip(rows[0], r)) for r in rows[2:]], dict(zip(rows[0], rows[1]))


# ---- launch list
lpath = os.path.join(src, f"launches_{tag}.csv")
if os.path.exists(lpath):
    lines = open(lpath).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
    per = defaultdict(list)
    for r in rows:
        if r.get("Metric Name") == "gpu__time_duration.sum":
            name = r["Kernel Name"].split("(")[0].replace("void ", "").split("<")[0]
            v = float(r["Metric Value"].replace(",", ""))
            unit = r.get("Metric Unit", "ns")
            per[name].append(v / 1e3 if unit == "ns" else v)  # -> us
    tot = sum(sum(v) for v in per.values())
    with open(os.path.join(out, f"{tag}_launches.txt"), "w") as f:
        f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none, command: "
                f"python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu --no-latency (C5, tcgen05 f16)\n")
        f.write("# kernel, launches, total us, mean us, share of all launched time\n")
        for name, v in sorted(per.items(), key=lambda x: -sum(x[1])):
            f.write(f"{name:40s} {len(v):4d} {sum(v):12.1f} {sum(v)/len(v):10.1f} {100*sum(v)/tot:6.2f}%\n")
    print(open(os.path.join(out, f"{tag}_launches.txt")).read())

traffic = {}
tj = os.path.join(out, "traffic.json")
if os.path.exists(tj):
    traffic = json.load(open(tj))
KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__bytes_read.sum.per_second",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active"]
for kind, key in (("tc", "C5_f16_g1"), ("fp32", "C3_fp32_g1"), ("dig", None),
                  ("fammllb", "FAM_mllb_g1"), ("famkml", "FAM_kml_g1"), ("scatter", None),
                  ("nn", None)):
    rep = os.path.join(src, f"full_{kind}_{tag}.ncu-rep")
    if not os.path.exists(rep):
        continue
    ms, units = raw_metrics(rep)
    m = ms[0]
    lines = [f"# ncu --set full --clock-control none --import-source on, report {os.path.basename(rep)}",
             f"# kernel: {m.get('Kernel Name', '')[:120]}"]
    for k in KEYS:
        if k in m:
            lines.append(f"{k:70s} {m[k]:>16s} {units.get(k, '')}")
    stalls = [(k, float(v or 0)) for k, v in m.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")]
    tot = sum(v for _, v in stalls) or 1
    lines.append("# warp-stall sampling (share of samples)")
    for k, v in sorted(stalls, key=lambda x: -x[1])[:8]:
        lines.append(f"  {k[33:]:30s} {100 * v / tot:5.1f}%")
    try:
        lines.append("# top source lines")
        sl = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "ncu_lines.py"), rep, "15"],
                            capture_output=True, text=True).stdout
        lines += ["  " + l for l in sl.splitlines()]
    except Exception:
        pass
    with open(os.path.join(out, f"{tag}_{kind}_full.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines[:20]))
    if key:
        def num(k):
            v = m.get(k, "0").replace(",", "")
            u = units.get(k, "byte")
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            return float(v) * scale
        traffic[key] = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
with open(tj, "w") as f:
    json.dump(traffic, f, indent=1, sort_keys=True)
print("traffic:", traffic)
