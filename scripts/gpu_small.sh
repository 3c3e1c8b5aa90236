#!/bin/bash
# small-batch latency probe: host path per batch size, NN/NN+2, fp32/f16
cat > /tmp/small.py <<'PY'
import time, numpy as np, torch, sys, os
sys.path.insert(0, os.getcwd())
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake
torch.cuda.set_device(0)
raw_all = inputs.device_trace("azure", 4096, 1200, 1.0)["raw"]
s = torch.cuda.current_stream()
for arch in (0, 2):
    lake.load_weights(40 + arch, arch, inputs.weights(arch, 0), 0)
    for prec in ("fp32", "f16"):
        flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
        for b in (1, 8, 64, 512, 4096):
            raw = np.ascontiguousarray(raw_all[:b])
            h_in = torch.from_numpy(raw.view(np.int32)).pin_memory()
            h_dec = torch.empty(b, dtype=torch.uint8).pin_memory()
            stb = lake.host_staging_bytes(b, flags)
            stg = torch.empty(stb, dtype=torch.uint8, device="cuda")
            for _ in range(50):
                lake.infer_host(h_in, flags, b, 40 + arch, None, h_dec, None, stg, stb, s)
            ts = []
            for _ in range(300):
                t0 = time.perf_counter(); lake.infer_host(h_in, flags, b, 40 + arch, None, h_dec, None, stg, stb, s); ts.append((time.perf_counter() - t0) * 1e6)
            print(arch, prec, b, "median us", round(float(np.median(ts)), 2), "p99", round(float(np.percentile(ts, 99)), 2), flush=True)
PY
timeout 300 python /tmp/small.py > gpurun_out/small_${1:-x}.txt 2>&1
