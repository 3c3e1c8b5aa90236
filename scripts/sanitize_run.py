"""Small invocation of every kernel, for compute-sanitizer:
digitise, FP32 (16- and 64-row tiles), tcgen05 fp16/bf16, multi-model grouping, capture,
host pipeline (zero-copy + chunked), persistent server."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake  # noqa: E402

torch.cuda.set_device(0)
dev = "cuda:0"
raw = inputs.edge_raw(3000, seed=1)
x = torch.from_numpy(raw.view(np.int32)).to(dev)
for m, a in ((1, 0), (2, 1), (3, 2)):
    lake.load_weights(m, a, inputs.weights(a, m), 0)
d = torch.empty((3000, 32), dtype=torch.uint8, device=dev)
lake.digitize(x, 129, d)
dec = torch.empty(3000, dtype=torch.uint8, device=dev)
lg = torch.empty((3000, 2), dtype=torch.float32, device=dev)
for n in (1, 129, 3000):
    for f in (lake.LAKE_PREC_FP32, lake.LAKE_PREC_F16, lake.LAKE_PREC_BF16):
        lake.infer(x, lake.LAKE_IN_RAW | f, n, 3, dec, lg)
lake.infer(d, lake.LAKE_IN_DIGITS | lake.LAKE_PREC_F16, 129, 2, dec, lg)
# NN kernel (output layer on the tensor cores) and tf32
for n in (1, 129, 3000):
    for f in (lake.LAKE_PREC_F16, lake.LAKE_PREC_BF16):
        lake.infer(x, lake.LAKE_IN_RAW | f, n, 1, dec, lg)
    lake.infer(x, lake.LAKE_IN_RAW | lake.LAKE_PREC_TF32, n, 3, dec, lg)
lake.infer(d, lake.LAKE_IN_DIGITS | lake.LAKE_PREC_F16, 3000, 1, dec, lg)
ids = torch.from_numpy(np.random.default_rng(0).integers(1, 4, 3000).astype(np.int32)).to(dev)
wsb = lake.workspace_bytes(3000)
ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
lake.infer_multi(x, lake.LAKE_IN_RAW | lake.LAKE_PREC_F16, 3000, ids, dec, lg, ws, wsb)
lake.infer_multi(x, lake.LAKE_IN_RAW | lake.LAKE_PREC_FP32, 3000, ids, dec, lg, ws, wsb)
lake.infer_multi(x, lake.LAKE_IN_RAW | lake.LAKE_PREC_TF32, 3000, ids, dec, lg, ws, wsb)
ids1 = torch.ones(3000, dtype=torch.int32, device=dev)  # NN only: one NN-layout kernel
lake.infer_multi(x, lake.LAKE_IN_RAW | lake.LAKE_PREC_F16, 3000, ids1, dec, lg, ws, wsb)
tr = inputs.device_trace("azure", 1000, 3, 3.0)
a = torch.from_numpy(tr["arrival_ns"]).to(dev)
c = torch.from_numpy(tr["complete_ns"]).to(dev)
out = torch.empty((1000, 9), dtype=torch.int32, device=dev)
cwb = lake.capture_workspace_bytes(1000)
cws = torch.empty(cwb, dtype=torch.uint8, device=dev)
lake.capture(a, c, None, 1000, out, cws, cwb)
h_in = torch.from_numpy(raw.view(np.int32)).pin_memory()
h_dec = torch.empty(3000, dtype=torch.uint8).pin_memory()
sb = lake.host_staging_bytes(3000, lake.LAKE_IN_RAW)
stg = torch.empty(sb, dtype=torch.uint8, device=dev)
lake.infer_host(h_in, lake.LAKE_IN_RAW | lake.LAKE_PREC_F16, 3000, 3, None, h_dec, None, stg, sb)
# one-byte model ids through the host path; NEXT-4 MLP family (fixed-shape and generic
# kernels, aligned bulk-copy staging and unaligned cp.async staging, ragged tiles)
h_ids8 = torch.from_numpy(np.random.default_rng(1).integers(1, 4, 3000).astype(np.uint8)).pin_memory()
lake.infer_host(h_in, lake.LAKE_IN_RAW | lake.LAKE_PREC_F16 | lake.LAKE_IDS_U8, 3000, -1, h_ids8,
                h_dec, None, stg, sb)
from paper_conf_asplos_finglertyshar23_b200.inputs import family  # noqa: E402
for mid, (shape, act) in enumerate((((15, 10, 10, 2), 0), ((5, 15, 15, 4), 1), ((16, 8, 5), 0))):
    lake.mlp_load(mid, shape, act, family.weights(shape, mid), 0)
    fx = torch.from_numpy(family.features(40001, shape[0], mid)).to(dev)
    cls = torch.empty(40001, dtype=torch.int32, device=dev)
    fo = torch.empty((40001, shape[-1]), dtype=torch.float32, device=dev)
    for n in (1, 129, 40001):
        lake.mlp_infer(fx, n, mid, cls, fo)
    flat = fx.flatten()
    lake.mlp_infer(flat[1:1 + 999 * shape[0]], 999, mid, cls, fo)  # 4-byte aligned only
    prev = lake.mlp_force_generic(True)
    lake.mlp_infer(fx, 40001, mid, cls, None)
    lake.mlp_force_generic(prev)
torch.cuda.synchronize()
if os.environ.get("SANITIZE_SERVER", "1") == "1":
    with lake.Server(3) as srv:
        hd = np.zeros(64, np.uint8)
        srv.infer(np.ascontiguousarray(raw[:5]), 5, hd)
        srv.infer(np.ascontiguousarray(raw[:64]), 64, hd)
torch.cuda.synchronize()
print("sanitize run ok")
if os.environ.get("LAKE_SAN_BIG"):
    # more 4,096-I/O chunks than scatter blocks (one per SM): every block streams several
    # chunks through its bulk-copy ring (next-chunk histogram loads and reservations)
    nb = 148 * 4096 * 2 + 777
    rawb = inputs.edge_raw(nb, seed=2)
    xb = torch.from_numpy(rawb.view(np.int32)).to(dev)
    idsb = torch.from_numpy(np.random.default_rng(1).integers(1, 4, nb).astype(np.int32)).to(dev)
    decb = torch.empty(nb, dtype=torch.uint8, device=dev)
    wsbb = lake.workspace_bytes(nb)
    wsb_t = torch.empty(wsbb, dtype=torch.uint8, device=dev)
    lake.multi_group(nb, idsb, wsb_t, wsbb)
    lake.infer_multi(xb, lake.LAKE_IN_RAW | lake.LAKE_PREC_F16, nb, idsb, decb, None, wsb_t, wsbb)
    torch.cuda.synchronize()
    print("big multi ok")
