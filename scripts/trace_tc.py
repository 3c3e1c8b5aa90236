"""Timeline of the tcgen05 kernel from the trace build (make trace): clock64 stamps of the
MMA thread, two epilogue warps and the digitiser of the leader CTA of cluster 0.
usage: LAKE_LINNOS_LIB=build/trace/liblake_linnos_trace.so python scripts/trace_tc.py"""
import ctypes
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

KIND = {1: "XFULL", 2: "TEMPTY", 3: "HREADY", 4: "COMMIT", 5: "DFULL", 6: "CHUNK",
        7: "LAYEREND", 8: "XEMPTY", 9: "XARRIVE", 10: "ISSUED", 11: "LDWAIT", 12: "STS",
        13: "FENCE", 14: "TOP", 15: "SCHED", 16: "WREADY", 17: "MMA0", 18: "CX", 19: "O_HDONE",
        20: "O_COMMIT", 21: "E_HDONE", 22: "E_DOUT", 23: "E_TEMPTY"}
STREAM = ({0: "mma", 1: "dig0", 2: "dig1", 3: "epi3"} if os.environ.get("LAKE_TRACE_DIG") else
          {0: "mma", 1: "g0pl", 2: "g1pl", 3: "dig"} if os.environ.get("LAKE_TRACE_OTC") else
          {0: "mma", 1: "e3r1", 2: "e3r2", 3: "e7r1"} if os.environ.get("LAKE_TRACE_PAIR") else {0: "q0w4", 1: "q1w5", 2: "q2w6", 3: "q3w3"} if os.environ.get("LAKE_TRACE_QUAD") else {0: "mma", 1: "epi4", 2: "epi11", 3: "dig"})
CAP = int(os.environ.get("LAKE_TRACE_CAP", 1 << 16))  # 512 for the SMEM-log build (-DLAKE_TRACE_SMEM)

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
prec = sys.argv[2] if len(sys.argv) > 2 else "f16"
torch.cuda.set_device(0)
w = inputs.workload(cfg, arch=int(sys.argv[3]) if len(sys.argv) > 3 else None)
for m, (a, blob) in w["models"].items():
    lake.load_weights(m, a, blob, 0)
n = w["raw"].shape[0]
x = torch.from_numpy(w["raw"].view(np.int32)).cuda()
ids = torch.from_numpy(w["model_ids"]).cuda()
dec = torch.empty(n, dtype=torch.uint8, device="cuda")
wsb = lake.workspace_bytes(n)
ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
single = len(w["models"]) == 1  # single-model configs: lake_linnos_infer (staged raw rows)
mid0 = next(iter(w["models"]))
def call():
    if single:
        lake.infer(x, flags, n, mid0, dec, None)
    else:
        lake.infer_multi(x, flags, n, ids, dec, None, ws, wsb)
call()  # warm
L = lake.lib()
buf = torch.zeros(4 * CAP * 2, dtype=torch.int64, device="cuda")
L.lake_trace_set(ctypes.c_void_p(buf.data_ptr()))
torch.cuda.synchronize()
call()
torch.cuda.synchronize()
L.lake_trace_set(ctypes.c_void_p(0))
ev = buf.cpu().numpy().view(np.uint64).reshape(4, CAP, 2)
rows = []
for st in range(4):
    k = ev[st, :, 0]
    used = k != 0
    for key, c in zip(k[used], ev[st, used, 1]):
        rows.append((int(c), st, int(key >> 56), int((key >> 24) & 0xFFFFFFFF), int((key >> 8) & 0xFFFF), int(key & 0xFF)))
rows.sort()
clk = np.array([r[0] for r in rows])
tiles = max(r[3] for r in rows) + 1
print(f"events {len(rows)}, tiles in cluster 0: {tiles}, span {clk[-1] - clk[0]} cycles, {(clk[-1] - clk[0]) / tiles:.0f} cycles/tile")
c0 = np.array([r[0] for r in rows if (r[2] == 4 and r[4] == 0) or (r[2] == 5 and r[4] == 0 and r[1] == 0)])
d = np.diff(np.sort(c0))
if d.size:
    print(f"tile period (L0 commits): median {np.median(d):.0f} p10 {np.percentile(d, 10):.0f} p90 {np.percentile(d, 90):.0f}")
present = sorted(set(r[3] for r in rows))
mid = present[len(present) // 2 - 1] if len(present) > 2 else present[0]
sel = [r for r in rows if r[3] in (mid, mid + 1)]
base = sel[0][0]
for r in sel:
    print(f"  {r[0] - base:7d} {STREAM[r[1]]:5s} {KIND.get(r[2], r[2]):9s} tile {r[3]} layer {r[4]} c/w {r[5]}")
