"""C4 NN (3 per-SSD models, 2^22 I/Os) through infer_multi only, a few calls (for ncu launch lists):
python scripts/c4_multi_only.py [arch] [prec] [reps]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

arch = int(sys.argv[1]) if len(sys.argv) > 1 else 0
prec = sys.argv[2] if len(sys.argv) > 2 else "f16"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
torch.cuda.set_device(0)
n = 1 << 22
w = inputs.workload("C4", n=n, arch=arch)
x = torch.from_numpy(w["raw"].view(np.int32)).cuda()
ids = torch.from_numpy(w["model_ids"]).cuda()
dec = torch.empty(n, dtype=torch.uint8, device="cuda")
wsb = lake.workspace_bytes(n)
ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
for m, (a, blob) in w["models"].items():
    lake.load_weights(m, a, blob, 0)
flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
for _ in range(reps):
    lake.infer_multi(x, flags, n, ids, dec, None, ws, wsb)
torch.cuda.synchronize()
print("ok", ids.dtype)
