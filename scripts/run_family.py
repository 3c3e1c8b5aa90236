"""One 2^24-row lake_mlp_infer launch per NEXT-4 model (for ncu captures)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_finglertyshar23_b200 import lake  # noqa: E402
from paper_conf_asplos_finglertyshar23_b200.inputs import family  # noqa: E402

torch.cuda.set_device(0)
n = 1 << 24
for mid, name in enumerate(sys.argv[1:] or ["mllb", "kml"]):
    cfg = family.FAMILY[name]
    lake.mlp_load(mid, cfg["widths"], cfg["act"], family.weights(cfg["widths"], 0), 0)
    x = torch.from_numpy(family.features(n, cfg["widths"][0], 5)).cuda()
    c = torch.empty(n, dtype=torch.int32, device="cuda")
    for _ in range(2):
        lake.mlp_infer(x, n, mid, c)
    torch.cuda.synchronize()
    print(name, "ok")
