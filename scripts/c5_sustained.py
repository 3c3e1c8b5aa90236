"""C5 step (bench.py's infer_multi over 2^24 I/Os, 64 NN+2 models, fp16) run N times back to
back, each step timed with CUDA events; NVML SM clock, power, temperature and clock-event
reasons sampled between steps. Shows whether longer runs slow down (power/thermal) or not:
python scripts/c5_sustained.py [steps]"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402
import pynvml  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 100
torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
w = inputs.workload("C5")
n = w["raw"].shape[0]
for m, (a, blob) in w["models"].items():
    lake.load_weights(m, a, blob, 0)
xs = [torch.from_numpy(w["raw"].view(np.int32)).to(dev) for _ in range(2)]
ids = torch.from_numpy(w["model_ids"]).to(dev)
dec = torch.empty(n, dtype=torch.uint8, device=dev)
wsb = lake.workspace_bytes(n)
ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
flags = lake.LAKE_IN_RAW | lake.LAKE_PREC_F16
s = torch.cuda.current_stream()
evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
for i in range(3):
    lake.infer_multi(xs[i % 2], flags, n, ids, dec, None, ws, wsb, s)
torch.cuda.synchronize()
samples = []
import threading
import time
stop = threading.Event()


def sampler():
    t0 = time.time()
    while not stop.is_set():
        samples.append(dict(t_ms=round((time.time() - t0) * 1e3, 1),
                            sm_mhz=pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM),
                            mem_mhz=pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_MEM),
                            power_w=pynvml.nvmlDeviceGetPowerUsage(h) / 1000,
                            temp_c=pynvml.nvmlDeviceGetTemperature(h, pynvml.NVML_TEMPERATURE_GPU),
                            reasons=int(pynvml.nvmlDeviceGetCurrentClocksEventReasons(h))))
        time.sleep(0.02)


th = threading.Thread(target=sampler)
th.start()
for i in range(steps):
    evs[i][0].record(s)
    lake.infer_multi(xs[i % 2], flags, n, ids, dec, None, ws, wsb, s)
    evs[i][1].record(s)
torch.cuda.synchronize()
stop.set()
th.join()
t = [a.elapsed_time(b) for a, b in evs]
blk_n = max(steps // 15, 1)
for blk in range(0, steps, blk_n):
    print(json.dumps(dict(steps=f"{blk}-{blk + blk_n - 1}", ms_mean=round(float(np.mean(t[blk:blk + blk_n])), 4))))
for smp in samples:
    print(json.dumps(smp))
