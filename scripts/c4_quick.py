"""C4 timings (3 per-SSD models, 2^22 I/Os): three pre-split single-model calls and one
infer_multi, per architecture and tensor-core type, plus a single-model 2^24 call
(profiling helper): python scripts/c4_quick.py [precs] [archs]"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

precs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["f16"]
archs = [int(a) for a in sys.argv[2].split(",")] if len(sys.argv) > 2 else [0, 1, 2]
torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream()


def timed(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(reps):
        fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


n = 1 << 22
for arch in archs:
    w = inputs.workload("C4", n=n, arch=arch)
    x = torch.from_numpy(w["raw"].view(np.int32)).to(dev)
    ids = torch.from_numpy(w["model_ids"]).to(dev)
    dec = torch.empty(1 << 24, dtype=torch.uint8, device=dev)
    wsb = lake.workspace_bytes(n)
    ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
    for m, (a, blob) in w["models"].items():
        lake.load_weights(m, a, blob, 0)
    mids = w["model_ids"]
    parts = [torch.from_numpy(np.ascontiguousarray(w["raw"][mids == m]).view(np.int32)).to(dev)
             for m in range(3)]
    big = torch.from_numpy(np.ascontiguousarray(np.tile(w["raw"], (4, 1))).view(np.int32)).to(dev)
    for prec in precs:
        flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
        t_multi = timed(lambda: lake.infer_multi(x, flags, n, ids, dec, None, ws, wsb, stream))
        t_split = timed(lambda: [lake.infer(p, flags, p.shape[0], m, dec, None, stream)
                                 for m, p in enumerate(parts)])
        t_big = timed(lambda: lake.infer(big, flags, 1 << 24, 0, dec, None, stream))
        print(json.dumps(dict(arch=arch, prec=prec, presplit_ms=round(t_split, 4),
                              multi_ms=round(t_multi, 4), single_2p24_ms=round(t_big, 4),
                              single_2p24_ginf_s=round((1 << 24) / t_big / 1e6, 2))), flush=True)
    for m in w["models"]:
        lake.unload(m, 0)
