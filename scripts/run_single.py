"""Single-model lake_linnos_infer on a BASELINE config (profiling helper):
python scripts/run_single.py CONFIG PREC ARCH [reps]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

cfg, prec, arch = sys.argv[1], sys.argv[2], int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
torch.cuda.set_device(0)
w = inputs.workload(cfg, arch=arch)
n = w["raw"].shape[0]
lake.load_weights(0, arch, w["models"][0][1], 0)
x = torch.from_numpy(w["raw"].view(np.int32)).cuda()
dec = torch.empty(n, dtype=torch.uint8, device="cuda")
flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for _ in range(2):
    lake.infer(x, flags, n, 0, dec, None)
e0.record()
for _ in range(reps):
    lake.infer(x, flags, n, 0, dec, None)
e1.record()
torch.cuda.synchronize()
print(f"{cfg} arch {arch} {prec} n={n}: {e0.elapsed_time(e1) / reps:.4f} ms per call")
