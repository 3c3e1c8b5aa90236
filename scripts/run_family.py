"""2^24-row lake_mlp_infer launches per NEXT-4 model: one pair for ncu captures, or with
--time, CUDA-event timing of 20 launches after 3 warm-ups (A/B of kernel variants)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_finglertyshar23_b200 import lake  # noqa: E402
from paper_conf_asplos_finglertyshar23_b200.inputs import family  # noqa: E402

args = [a for a in sys.argv[1:] if not a.startswith("--")]
timing = "--time" in sys.argv
torch.cuda.set_device(0)
n = 1 << 24
for mid, name in enumerate(args or ["mllb", "kml"]):
    cfg = family.FAMILY[name]
    lake.mlp_load(mid, cfg["widths"], cfg["act"], family.weights(cfg["widths"], 0), 0)
    x = torch.from_numpy(family.features(n, cfg["widths"][0], 5)).cuda()
    c = torch.empty(n, dtype=torch.int32, device="cuda")
    reps = 20 if timing else 2
    for _ in range(3 if timing else 0):
        lake.mlp_infer(x, n, mid, c)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        lake.mlp_infer(x, n, mid, c)
    e1.record()
    torch.cuda.synchronize()
    print(name, f"{e0.elapsed_time(e1) / reps:.4f} ms" if timing else "ok")
