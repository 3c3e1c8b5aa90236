"""Seeded synthetic inputs for the NEXT-4 MLP family (MLLB / KML shapes).

Holds none of the method's arithmetic: it draws feature rows and random-init weights.
PAPER.md gives neither the shapes nor the features of these models (§7.3 P:1471-1475,
§7.4); the shapes are readings R25-R28:

* ``mllb``: 15 per-task load-balancing features -> 10 -> 10 -> 2 (migrate / stay), ReLU.
* ``kml``:  5 per-process I/O-pattern features -> 15 -> 15 -> 4 readahead classes, sigmoid.

Features are z-scored inputs (both works normalise their features), drawn N(0, 1), with a
fraction of exact zeros and large outliers so ReLU zeroing and sigmoid saturation occur.
Weights ~ U(+-1/sqrt(fan_in)) (PyTorch nn.Linear default), PCG64 seed 9000 + model_id.
"""
from __future__ import annotations

import numpy as np

ACT_RELU, ACT_SIGMOID = 0, 1

FAMILY = {
    "mllb": dict(widths=(15, 10, 10, 2), act=ACT_RELU),
    "kml": dict(widths=(5, 15, 15, 4), act=ACT_SIGMOID),
}


def blob_floats(widths) -> int:
    return int(sum(widths[l + 1] * widths[l] + widths[l + 1] for l in range(len(widths) - 1)))


def weights(widths, model_id: int) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(9000 + model_id))
    parts = []
    for l in range(len(widths) - 1):
        k, nout = widths[l], widths[l + 1]
        bound = 1.0 / np.sqrt(k)
        parts.append(rng.uniform(-bound, bound, size=(nout, k)).ravel())
        parts.append(rng.uniform(-bound, bound, size=nout))
    return np.concatenate(parts).astype(np.float32)


def features(n: int, width: int, seed: int) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(seed))
    x = rng.standard_normal((n, width)).astype(np.float32)
    if n:
        m = rng.random((n, width))
        x[m < 0.02] = 0.0
        x[m > 0.995] *= 40.0
    return x
