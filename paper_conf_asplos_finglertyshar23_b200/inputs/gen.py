"""Seeded trace / raw-record / weight generators (no method arithmetic; see __init__)."""
from __future__ import annotations

import ctypes
import json
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SIM_SRC = os.path.join(_HERE, "tracesim.c")
_SIM_SO = os.path.join(_HERE, "libtracesim.so")
_CALIB = os.path.join(_HERE, "bout_calibration.json")

# Table 4: avg IOPS, avg read/write size (KB), min/max inter-arrival (us).
# Azure and Bing-I are already the paper's doubled ("rerated") traces.
PROFILES = {
    "azure": dict(iops=26_000.0, read_kb=30.0, write_kb=19.0, max_ia_us=324.0),
    "bing_i": dict(iops=4_800.0, read_kb=73.0, write_kb=59.0, max_ia_us=1_800.0),
    "cosmos": dict(iops=2_500.0, read_kb=657.0, write_kb=609.0, max_ia_us=1_600.0),
}
PROFILE_ORDER = ("azure", "bing_i", "cosmos")

# Silent parameters: device latency model and size spread.
SIZE_SIGMA_LOG = 1.0          # log-normal sigma of I/O size
READ_FRACTION = 2.0 / 3.0
CHANNELS = 8                  # FIFO channels per device
SERVICE_BASE_US = 20.0        # fixed service cost
SERVICE_US_PER_KB = 0.25      # transfer cost
SERVICE_JITTER_SIGMA = 0.3    # LogNormal(0, 0.3) multiplicative jitter
GC_ENTER_P = 1e-3             # two-state "GC" modulator: enter probability per I/O
GC_MEAN_STAY = 200.0          # mean stay in I/Os
GC_SLOWDOWN = 4.0             # service multiplier while in GC

ARCH_WIDTHS = {0: (31, 256, 2), 1: (31, 256, 256, 2), 2: (31, 256, 256, 256, 2)}

# BASELINE.json configs as concrete runs; sizes are powers of two (S24).
CONFIGS = {
    "C1": dict(arch=0, n=4_096, models=1, rerate=1.0),
    "C2": dict(arch=None, n=4_096, models=1, rerate=1.0),
    "C3": dict(arch=2, n=1 << 20, models=1, rerate=1.0),
    "C4": dict(arch=2, n=1 << 22, models=3, rerate=3.0),
    "C5": dict(arch=2, n=1 << 24, models=64, rerate=3.0),
}


def blob_floats(arch: int) -> int:
    w = ARCH_WIDTHS[arch]
    return int(sum(w[i + 1] * w[i] + w[i + 1] for i in range(len(w) - 1)))


# --------------------------------------------------------------------------- tracesim
_sim = None


def _build_sim() -> str:
    if not os.path.exists(_SIM_SO) or os.path.getmtime(_SIM_SO) < os.path.getmtime(_SIM_SRC):
        subprocess.check_call(["gcc", "-std=gnu99", "-O2", "-shared", "-fPIC", "-o", _SIM_SO,
                               _SIM_SRC])
    return _SIM_SO


def _load_sim():
    global _sim
    if _sim is None:
        lib = ctypes.CDLL(_build_sim())
        P = ctypes.c_void_p
        lib.tracesim_run.argtypes = [P, P, ctypes.c_int64, ctypes.c_int, P, P]
        lib.tracesim_run.restype = ctypes.c_int
        lib.tracesim_markov.argtypes = [P, ctypes.c_int64, ctypes.c_double, ctypes.c_double, P]
        lib.tracesim_markov.restype = None
        _sim = lib
    return _sim


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def device_trace(profile: str, n: int, seed: int, rerate: float = 1.0,
                 t0_ns: int = 0) -> dict:
    """One device's trace: n I/Os, arrival-ordered. Returns dict with raw uint32[n, 9]
    (lake_io_raw_t layout), arrival_ns, complete_ns, size_kb, is_read, gc."""
    prof = PROFILES[profile]
    rng = np.random.Generator(np.random.PCG64(seed))
    mean_ia_us = 1e6 / (prof["iops"] * rerate)
    max_ia_us = prof["max_ia_us"] / rerate
    ia_us = np.minimum(rng.exponential(mean_ia_us, size=n), max_ia_us)
    is_read = rng.random(n) < READ_FRACTION
    mean_kb = np.where(is_read, prof["read_kb"], prof["write_kb"])
    mu = np.log(mean_kb) - 0.5 * SIZE_SIGMA_LOG ** 2
    size_kb = np.exp(mu + SIZE_SIGMA_LOG * rng.standard_normal(n))
    offset = rng.random(n)  # uniform offset; unused by the features  # noqa
    jitter = np.exp(SERVICE_JITTER_SIGMA * rng.standard_normal(n))
    u_gc = rng.random(n)
    gc = np.zeros(n, dtype=np.uint8)
    lib = _load_sim()
    if n:
        lib.tracesim_markov(_p(u_gc), n, GC_ENTER_P, 1.0 / GC_MEAN_STAY, _p(gc))
    service_us = (SERVICE_BASE_US + SERVICE_US_PER_KB * size_kb) * jitter
    service_us = service_us * np.where(gc == 1, GC_SLOWDOWN, 1.0)
    arrival_ns = t0_ns + np.cumsum(np.round(ia_us * 1000.0).astype(np.int64))
    service_ns = np.maximum(np.round(service_us * 1000.0).astype(np.int64), 1)
    complete_ns = np.zeros(n, dtype=np.int64)
    raw = np.zeros((n, 9), dtype=np.uint32)
    if n:
        rc = lib.tracesim_run(_p(arrival_ns), _p(service_ns), n, CHANNELS, _p(complete_ns),
                              _p(raw))
        if rc != 0:
            raise MemoryError("tracesim_run failed")
    return dict(raw=raw, arrival_ns=arrival_ns, complete_ns=complete_ns, size_kb=size_kb,
                is_read=is_read, gc=gc)


def multi_device_trace(n_total: int, n_devices: int, seed_base: int, rerate: float = 3.0):
    """Interleave n_devices per-SSD streams by arrival time (mixed workload).
    Device d uses profile PROFILE_ORDER[d % 3] and model id d; per-device I/O counts are
    proportional to each profile's rerated IOPS so the streams span the same time window.
    Returns (raw uint32[n_total, 9], model_ids int32[n_total])."""
    iops = np.array([PROFILES[PROFILE_ORDER[d % 3]]["iops"] for d in range(n_devices)])
    share = iops / iops.sum() * n_total
    counts = np.floor(share).astype(np.int64)
    rem = n_total - int(counts.sum())
    order = np.argsort(-(share - counts), kind="stable")
    counts[order[:rem]] += 1
    raws, arrs, mids = [], [], []
    for d in range(n_devices):
        tr = device_trace(PROFILE_ORDER[d % 3], int(counts[d]), seed_base + d, rerate)
        raws.append(tr["raw"])
        arrs.append(tr["arrival_ns"])
        mids.append(np.full(int(counts[d]), d, dtype=np.int32))
    raw = np.concatenate(raws) if raws else np.zeros((0, 9), np.uint32)
    arr = np.concatenate(arrs) if arrs else np.zeros(0, np.int64)
    mid = np.concatenate(mids) if mids else np.zeros(0, np.int32)
    perm = np.lexsort((mid, arr))  # by arrival, ties by device id
    return np.ascontiguousarray(raw[perm]), np.ascontiguousarray(mid[perm])


# --------------------------------------------------------------------------- weights
def raw_weights(arch: int, model_id: int) -> np.ndarray:
    """Random init like torch.nn.Linear: W, b ~ U(+-1/sqrt(fan_in)), PCG64(7000+model_id).
    Blob layout = lake_linnos_load_weights: per layer W[out][in] then b[out]."""
    w = ARCH_WIDTHS[arch]
    rng = np.random.Generator(np.random.PCG64(7000 + int(model_id)))
    parts = []
    for l in range(len(w) - 1):
        fan_in, fan_out = w[l], w[l + 1]
        bound = 1.0 / np.sqrt(fan_in)
        parts.append(rng.uniform(-bound, bound, size=fan_out * fan_in).astype(np.float32))
        parts.append(rng.uniform(-bound, bound, size=fan_out).astype(np.float32))
    blob = np.concatenate(parts)
    assert blob.size == blob_floats(arch)
    return blob


_calib_cache = None


def _calibration() -> dict:
    global _calib_cache
    if _calib_cache is None:
        if os.path.exists(_CALIB):
            with open(_CALIB) as f:
                _calib_cache = json.load(f)["bout"]
        else:
            _calib_cache = {}
    return _calib_cache


def weights(arch: int, model_id: int, calibrated: bool = True) -> np.ndarray:
    """raw_weights with the output bias replaced by the stored re-centred value, so that
    decisions are ~50/50 slow/fast. The stored values were written by
    scripts/calibrate_bout.py, which calls only oracle/."""
    blob = raw_weights(arch, model_id)
    if calibrated:
        key = f"arch{arch}_model{model_id}"
        c = _calibration().get(key)
        if c is not None:
            blob[-2:] = np.array([int(h, 16) for h in c], dtype=np.uint32).view(np.float32)
    return blob


# --------------------------------------------------------------------------- edge cases
EDGE_VALUES = np.array([0, 1, 9, 10, 99, 100, 999, 1000, 1001, 9998, 9999, 10000, 10001,
                        65535, 65536, 99999, 100000, 2**31 - 1, 2**31, 2**32 - 1],
                       dtype=np.uint64)


def edge_raw(n: int, seed: int) -> np.ndarray:
    """Adversarial raw records: a mix of digit-boundary values and uniform uint32 / small
    values, for bit-exact digitisation and saturation coverage."""
    rng = np.random.Generator(np.random.PCG64(seed))
    kind = rng.integers(0, 3, size=(n, 9))
    edge = EDGE_VALUES[rng.integers(0, EDGE_VALUES.size, size=(n, 9))]
    small = rng.integers(0, 20_000, size=(n, 9), dtype=np.uint64)
    full = rng.integers(0, 2**32, size=(n, 9), dtype=np.uint64)
    out = np.where(kind == 0, edge, np.where(kind == 1, small, full))
    return np.ascontiguousarray(out.astype(np.uint32))


# --------------------------------------------------------------------------- configs
def workload(name: str, n: int | None = None, arch: int | None = None):
    """Inputs of a BASELINE config. Returns dict(raw, model_ids, models={id: (arch, blob)}).
    Trace seed = 1000 + 100*config_index (+ device)."""
    cfg = CONFIGS[name]
    ci = int(name[1:])
    n = cfg["n"] if n is None else int(n)
    arch = cfg["arch"] if arch is None else arch
    if arch is None:
        arch = 0
    seed = 1000 + 100 * ci
    if cfg["models"] == 1:
        tr = device_trace("azure", n, seed, cfg["rerate"])
        raw = tr["raw"]
        mids = np.zeros(n, dtype=np.int32)
    else:
        raw, mids = multi_device_trace(n, cfg["models"], seed, cfg["rerate"])
    models = {m: (arch, weights(arch, m)) for m in range(cfg["models"])}
    return dict(raw=raw, model_ids=mids, models=models, arch=arch)
