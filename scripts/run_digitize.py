"""Launch the standalone digitise kernel on a C5-sized batch (2^24 raw records) once, for
ncu capture and a quick device-time measurement."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

n = 1 << 24
raw = inputs.edge_raw(1 << 20, seed=1)
raw = np.tile(raw, (16, 1))
x = torch.from_numpy(raw.view(np.int32)).cuda()
d = torch.empty((n, 32), dtype=torch.uint8, device="cuda")
lake.digitize(x, n, d)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    lake.digitize(x, n, d)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 10
print(f"digitize n={n}: {ms:.3f} ms, {n * 68 / ms / 1e6:.1f} GB/s algorithmic (68 B/IO)")
