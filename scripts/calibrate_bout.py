"""Write paper_conf_asplos_finglertyshar23_b200/inputs/bout_calibration.json.

Re-centres each random-init model's output bias so that its decisions are ~50/50
slow/fast on a calibration trace (reading R16): without it one seed gave
99.9% "slow" and every agreement test would be vacuous. Calls ONLY oracle/ (plus the
seeded generators); no value here comes from the CUDA path.

    margin_i = logit1_i - logit0_i      (oracle, float64 of the float32 logits)
    m        = median(margin)
    bout'    = float32(bout[0] + m/2), float32(bout[1] - m/2)

Calibration covers every model_id in [0, LAKE_MAX_MODELS), so a test may use any id.
Calibration trace per model: device profile PROFILE_ORDER[model % 3], rerate x3,
4096 I/Os, seed 555000 + model.
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_asplos_finglertyshar23_b200.inputs import gen  # noqa: E402

N_MODELS = 1024  # every model_id slot (LAKE_MAX_MODELS): tests may load any id
N_CAL = 4096


def main():
    out = {}
    for arch in (0, 1, 2):
        for m in range(N_MODELS):
            blob = gen.raw_weights(arch, m)
            raw = gen.device_trace(gen.PROFILE_ORDER[m % 3], N_CAL, 555000 + m, 3.0)["raw"]
            lg, _ = oracle.infer_raw(arch, blob, raw, nthreads=0)
            med = float(np.median(lg[:, 1].astype(np.float64) - lg[:, 0]))
            b = np.array([blob[-2] + med / 2, blob[-1] - med / 2], dtype=np.float32)
            out[f"arch{arch}_model{m}"] = [f"{v:08x}" for v in b.view(np.uint32)]
        print("arch", arch, "done", flush=True)
    path = os.path.join(ROOT, "paper_conf_asplos_finglertyshar23_b200", "inputs",
                        "bout_calibration.json")
    with open(path, "w") as f:
        json.dump({"method": __doc__.strip().splitlines()[2], "n_cal": N_CAL, "bout": out}, f,
                  indent=0, sort_keys=True)
    print("wrote", path)


if __name__ == "__main__":
    main()
