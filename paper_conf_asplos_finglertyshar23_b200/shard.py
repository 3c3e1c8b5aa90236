"""Placement of per-SSD models and their I/O streams across GPUs (host logic).

One feature registry — hence one model — per block device (Fig. 4 caption,
P:906-909), and each I/O's decision depends only on its own record and its device's model,
so the batch shards with no collective on the data path. Two plans:

* ``model_affine``: every model lives on exactly one rank; models are assigned
  longest-processing-time first (largest I/O count to the least-loaded rank, ties to the
  lower rank), so per-rank loads stay balanced even though Table 4's profiles differ 10x in
  IOPS. Each rank holds only its models' weights.
* ``range_split``: contiguous I/O ranges, all weights replicated on every rank (the
  balance fallback when one model dominates).

Both are deterministic functions of (counts, world); every rank computes the same plan.
"""
from __future__ import annotations

import numpy as np


def model_affine(counts: np.ndarray, world: int) -> np.ndarray:
    """counts[m] = I/Os of model m. Returns owner[m] in [0, world)."""
    counts = np.asarray(counts, dtype=np.int64)
    owner = np.zeros(counts.size, dtype=np.int64)
    load = np.zeros(world, dtype=np.int64)
    order = np.lexsort((np.arange(counts.size), -counts))  # count desc, then model id
    for m in order:
        r = int(np.argmin(load))  # first minimum -> lowest rank on ties
        owner[m] = r
        load[r] += counts[m]
    return owner


def imbalance(counts: np.ndarray, owner: np.ndarray, world: int) -> float:
    """max rank load / mean rank load (1.0 = perfect)."""
    load = np.bincount(owner, weights=np.asarray(counts, np.float64), minlength=world)
    return float(load.max() / max(load.mean(), 1e-12))


def rank_indices(model_ids: np.ndarray, owner: np.ndarray, rank: int) -> np.ndarray:
    """Positions (in arrival order) of the I/Os whose model is owned by `rank`."""
    mine = owner[np.asarray(model_ids, np.int64)] == rank
    return np.nonzero(mine)[0]


def range_split(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous [begin, end) of I/O positions for `rank` (sizes differ by at most 1)."""
    base, rem = divmod(n, world)
    begin = rank * base + min(rank, rem)
    return begin, begin + base + (1 if rank < rem else 0)


def plan(model_ids: np.ndarray, n_models: int, world: int, max_imbalance: float = 1.01):
    """Pick model-affine if it balances within max_imbalance, else range split.
    Returns dict(kind, owner or None, imbalance)."""
    counts = np.bincount(np.asarray(model_ids, np.int64), minlength=n_models)
    owner = model_affine(counts, world)
    imb = imbalance(counts, owner, world)
    if imb <= max_imbalance:
        return dict(kind="model_affine", owner=owner, imbalance=imb)
    return dict(kind="range_split", owner=None, imbalance=1.0)
