"""Timeline of the two-tile tcgen05 kernel (mlp_tc2.cu) from the trace build (make trace):
clock64 stamps of the MMA thread, epilogue warps 3 and 18 and digitiser thread 0 of the
leader CTA of cluster 0. usage:
  LAKE_LINNOS_LIB=build/trace/liblake_linnos_trace.so python scripts/trace_tc2.py [C5] [f16]"""
import ctypes
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

KIND = {1: "TEMPTY", 2: "XFULL", 3: "HFULL", 4: "DFULL", 5: "CONV", 6: "HFREE", 7: "LOGITS",
        8: "GATHER", 9: "XEMPTY", 10: "XARRIVE"}
STREAM = {0: "mma", 1: "epi3", 2: "epi18", 3: "dig"}
CAP = 1 << 16
cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
prec = sys.argv[2] if len(sys.argv) > 2 else "f16"
torch.cuda.set_device(0)
w = inputs.workload(cfg)
for m, (a, blob) in w["models"].items():
    lake.load_weights(m, a, blob, 0)
n = w["raw"].shape[0]
x = torch.from_numpy(w["raw"].view(np.int32)).cuda()
ids = torch.from_numpy(w["model_ids"]).cuda()
dec = torch.empty(n, dtype=torch.uint8, device="cuda")
wsb = lake.workspace_bytes(n)
ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
lake.infer_multi(x, flags, n, ids, dec, None, ws, wsb)
L = lake.lib()
buf = torch.zeros(4 * CAP * 2, dtype=torch.int64, device="cuda")
L.lake_trace2_set(ctypes.c_void_p(buf.data_ptr()))
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
lake.infer_multi(x, flags, n, ids, dec, None, ws, wsb)
e1.record()
torch.cuda.synchronize()
print("traced launch ms", e0.elapsed_time(e1))
L.lake_trace2_set(ctypes.c_void_p(0))
ev = buf.cpu().numpy().view(np.uint64).reshape(4, CAP, 2)
rows = []
for st in range(4):
    k = ev[st, :, 0]
    used = k != 0
    for key, c in zip(k[used], ev[st, used, 1]):
        rows.append((int(c), st, int(key >> 56), int((key >> 24) & 0xFFFFFFFF),
                     int((key >> 8) & 0xFFFF), int(key & 0xFF)))
rows.sort()
clk = np.array([r[0] for r in rows])
print(f"events {len(rows)}, span {clk[-1] - clk[0]} cycles")
xf = np.array([r[0] for r in rows if r[1] == 0 and r[2] == 2])
d = np.diff(xf)
print(f"L0 starts (XFULL ok): {len(xf)}, period per tile median {np.median(d):.0f} "
      f"(pairs: {np.median(d[::2]):.0f} / {np.median(d[1::2]):.0f})")
mid = len(xf) // 2
t0, t1 = xf[mid], xf[mid + 4]
for r in rows:
    if t0 - 200 <= r[0] <= t1:
        print(f"  {r[0] - t0:7d} {STREAM[r[1]]:5s} {KIND.get(r[2], r[2]):8s} tile {r[3]} layer {r[4]} x {r[5]}")
