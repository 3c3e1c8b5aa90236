"""GPU feature-capture timing (lake_linnos_capture over a synthetic single-device trace):
python scripts/capture_time.py [log2 n ...]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

torch.cuda.set_device(0)
for lg in [int(x) for x in sys.argv[1:]] or [20, 24]:
    n = 1 << lg
    tr = inputs.device_trace("azure", n, 3, 3.0)
    a = torch.from_numpy(tr["arrival_ns"]).cuda()
    c = torch.from_numpy(tr["complete_ns"]).cuda()
    out = torch.empty((n, 9), dtype=torch.int32, device="cuda")
    cwb = lake.capture_workspace_bytes(n)
    cws = torch.empty(cwb, dtype=torch.uint8, device="cuda")
    for _ in range(2):
        lake.capture(a, c, None, n, out, cws, cwb)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5):
        lake.capture(a, c, None, n, out, cws, cwb)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    print(f"capture n=2^{lg}: {ms:.3f} ms = {n / ms / 1e6:.2f} G records/s, workspace {cwb / 2**20:.0f} MiB")
