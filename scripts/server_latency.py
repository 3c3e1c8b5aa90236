"""Latency of the persistent doorbell server vs the launch-based host path, per batch size."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

torch.cuda.set_device(0)
raw_all = inputs.device_trace("azure", 4096, 1200, 1.0)["raw"]
for arch in (0, 1, 2):
    lake.load_weights(40 + arch, arch, inputs.weights(arch, 0), 0)
    with lake.Server(40 + arch) as srv:
        for b in (1, 4, 8, 16, 32, 64):
            raw = np.ascontiguousarray(raw_all[:b])
            dec = np.zeros(b, np.uint8)
            for _ in range(200):
                srv.infer(raw, b, dec)
            ts = []
            for _ in range(2000):
                t0 = time.perf_counter()
                srv.infer(raw, b, dec)
                ts.append((time.perf_counter() - t0) * 1e6)
            print(f"arch {arch} batch {b:3d} server median {np.median(ts):7.2f} us  p99 {np.percentile(ts, 99):7.2f} us", flush=True)

# phase breakdown of one batch (development hook)
import ctypes  # noqa: E402
L = lake.lib()
t = (ctypes.c_ulonglong * 8)()
for arch in (0, 2):
    lake.load_weights(40 + arch, arch, inputs.weights(arch, 0), 0)
    with lake.Server(40 + arch) as srv:
        for b in (1, 64):
            raw = np.ascontiguousarray(raw_all[:b])
            dec = np.zeros(b, np.uint8)
            for _ in range(100):
                srv.infer(raw, b, dec)
            L.lake_debug_server_times(srv._h, t)
            v = list(t)
            print(f"arch {arch} b {b}: digitise {(v[1]-v[0])/1e3:.2f} us, layers",
                  [round((v[2+l] - (v[1+l] if l else v[1]))/1e3, 2) for l in range(arch + 1)],
                  f"out {(v[5]-v[2+arch])/1e3:.2f} us, fence {(v[6]-v[5])/1e3:.2f} us", flush=True)
