"""CPU oracle for the batched LinnOS classifier — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package. The product package
(``paper_conf_asplos_finglertyshar23_b200``) never imports it and shares no code with it.

This module is argument marshalling (numpy <-> ctypes) around ``lake_oracle.c``, which
holds all the arithmetic, written from the paper (see that file's header for the
citations and readings). Parity status per function:

* ``digitize``              pinned (hand-worked golden examples, brute-force round trip)
* ``mlp`` / ``infer_raw``   pinned (tiny integer MLPs vs int64, IEEE order examples,
                             invariants, numpy float64 GEMM chain)
* ``capture``               pinned (hand-worked trace, heap-based event simulation of the
                             generator, invariants)
* ``mlp_family``            pinned (NEXT-4: tiny integer ReLU MLPs vs int64 with C = 4
                             and first-max ties, sigmoid special values and a float64
                             chain, NaN / tie class rules, C = 2 against ``mlp``)
* parity against the paper's trained model: unpinned (no weights/traces published).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liblake_oracle.so")
_SRC = os.path.join(_HERE, "lake_oracle.c")

CFLAGS = ["-std=gnu99", "-O2", "-mfma", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
          "-shared", "-fPIC"]

ARCH_WIDTHS = {0: (31, 256, 2), 1: (31, 256, 256, 2), 2: (31, 256, 256, 256, 2)}


def build(force: bool = False) -> str:
    """Compile lake_oracle.c into liblake_oracle.so (gcc). Returns the .so path."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, "-o", _SO, _SRC, "-lm"])
    return _SO


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        lib.oracle_digitize.argtypes = [P, ctypes.c_int64, P]
        lib.oracle_digitize.restype = None
        lib.oracle_mlp.argtypes = [ctypes.c_int, P, P, P, ctypes.c_int64, P, P, ctypes.c_int]
        lib.oracle_mlp.restype = ctypes.c_int
        lib.oracle_infer_raw.argtypes = [ctypes.c_int, P, P, ctypes.c_int64, P, P, ctypes.c_int]
        lib.oracle_infer_raw.restype = ctypes.c_int
        lib.oracle_infer_digits.argtypes = [ctypes.c_int, P, P, ctypes.c_int64, P, P,
                                            ctypes.c_int]
        lib.oracle_infer_digits.restype = ctypes.c_int
        lib.oracle_capture.argtypes = [P, P, P, ctypes.c_int64, P]
        lib.oracle_capture.restype = None
        lib.oracle_capture_rows.argtypes = [P, P, P, ctypes.c_int64, P, ctypes.c_int64, P]
        lib.oracle_capture_rows.restype = None
        lib.oracle_mlp_family.argtypes = [ctypes.c_int, P, ctypes.c_int, P, P, ctypes.c_int64,
                                          P, P, ctypes.c_int]
        lib.oracle_mlp_family.restype = ctypes.c_int
        lib.oracle_max_threads.argtypes = []
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def digitize(raw: np.ndarray) -> np.ndarray:
    """raw uint32[n, 9] -> digits uint8[n, 31]."""
    raw = np.ascontiguousarray(raw, dtype=np.uint32).reshape(-1, 9)
    out = np.zeros((raw.shape[0], 31), dtype=np.uint8)
    _load().oracle_digitize(_ptr(raw), raw.shape[0], _ptr(out))
    return out


def mlp(widths, blob: np.ndarray, x: np.ndarray, nthreads: int = 1):
    """Generic strict-order FP32 MLP. Returns (logits float32[n,2], decisions uint8[n])."""
    widths = np.ascontiguousarray(widths, dtype=np.int32)
    blob = np.ascontiguousarray(blob, dtype=np.float32)
    x = np.ascontiguousarray(x, dtype=np.float32).reshape(-1, int(widths[0]))
    n = x.shape[0]
    logits = np.zeros((n, 2), dtype=np.float32)
    dec = np.zeros(n, dtype=np.uint8)
    rc = _load().oracle_mlp(len(widths) - 1, _ptr(widths), _ptr(blob), _ptr(x), n,
                            _ptr(logits), _ptr(dec), nthreads)
    if rc != 0:
        raise ValueError(f"oracle_mlp failed ({rc})")
    return logits, dec


def infer_raw(arch: int, blob: np.ndarray, raw: np.ndarray, nthreads: int = 1):
    """score_features on raw records: (logits float32[n,2], decisions uint8[n])."""
    blob = np.ascontiguousarray(blob, dtype=np.float32)
    raw = np.ascontiguousarray(raw, dtype=np.uint32).reshape(-1, 9)
    n = raw.shape[0]
    logits = np.zeros((n, 2), dtype=np.float32)
    dec = np.zeros(n, dtype=np.uint8)
    rc = _load().oracle_infer_raw(arch, _ptr(blob), _ptr(raw), n, _ptr(logits), _ptr(dec),
                                  nthreads)
    if rc != 0:
        raise ValueError(f"oracle_infer_raw failed ({rc})")
    return logits, dec


def infer_digits(arch: int, blob: np.ndarray, digits: np.ndarray, nthreads: int = 1):
    """score_features on digits uint8[n, 31] (or [n, 32]; the pad byte is dropped)."""
    blob = np.ascontiguousarray(blob, dtype=np.float32)
    d = np.asarray(digits, dtype=np.uint8)
    if d.ndim == 2 and d.shape[1] == 32:
        d = d[:, :31]
    d = np.ascontiguousarray(d).reshape(-1, 31)
    n = d.shape[0]
    logits = np.zeros((n, 2), dtype=np.float32)
    dec = np.zeros(n, dtype=np.uint8)
    rc = _load().oracle_infer_digits(arch, _ptr(blob), _ptr(d), n, _ptr(logits), _ptr(dec),
                                     nthreads)
    if rc != 0:
        raise ValueError(f"oracle_infer_digits failed ({rc})")
    return logits, dec


def infer_multi_raw(models: dict, raw: np.ndarray, model_ids: np.ndarray, nthreads: int = 1):
    """Per-model scoring of an interleaved batch: models = {model_id: (arch, blob)}.
    I/Os whose model id is unknown get decision 0 and NaN logits (header contract)."""
    raw = np.ascontiguousarray(raw, dtype=np.uint32).reshape(-1, 9)
    model_ids = np.asarray(model_ids, dtype=np.int32)
    n = raw.shape[0]
    logits = np.full((n, 2), np.nan, dtype=np.float32)
    dec = np.zeros(n, dtype=np.uint8)
    for mid, (arch, blob) in models.items():
        idx = np.nonzero(model_ids == mid)[0]
        if idx.size == 0:
            continue
        lg, d = infer_raw(arch, blob, raw[idx], nthreads)
        logits[idx] = lg
        dec[idx] = d
    return logits, dec


ACT_RELU, ACT_SIGMOID = 0, 1


def mlp_family(widths, act: int, blob: np.ndarray, x: np.ndarray, nthreads: int = 1):
    """NEXT-4 MLP family (MLLB / KML shapes): (out float32[n, C], classes int32[n])."""
    widths = np.ascontiguousarray(widths, dtype=np.int32)
    blob = np.ascontiguousarray(blob, dtype=np.float32)
    x = np.ascontiguousarray(x, dtype=np.float32).reshape(-1, int(widths[0]))
    n, C = x.shape[0], int(widths[-1])
    out = np.zeros((n, C), dtype=np.float32)
    cls = np.full(n, -1, dtype=np.int32)
    rc = _load().oracle_mlp_family(len(widths) - 1, _ptr(widths), act, _ptr(blob), _ptr(x), n,
                                   _ptr(out), _ptr(cls), nthreads)
    if rc != 0:
        raise ValueError(f"oracle_mlp_family failed ({rc})")
    return out, cls


def capture(arrival_ns: np.ndarray, complete_ns: np.ndarray, device=None) -> np.ndarray:
    """Feature capture (NEXT-1): per-I/O raw records uint32[n, 9] from a trace."""
    a = np.ascontiguousarray(arrival_ns, dtype=np.int64)
    c = np.ascontiguousarray(complete_ns, dtype=np.int64)
    n = a.shape[0]
    out = np.zeros((n, 9), dtype=np.uint32)
    d = None if device is None else np.ascontiguousarray(device, dtype=np.int32)
    _load().oracle_capture(_ptr(a), _ptr(c), None if d is None else _ptr(d), n, _ptr(out))
    return out


def capture_rows(arrival_ns, complete_ns, device, rows) -> np.ndarray:
    """capture() for selected rows only (O(n) per row): uint32[len(rows), 9]."""
    a = np.ascontiguousarray(arrival_ns, dtype=np.int64)
    c = np.ascontiguousarray(complete_ns, dtype=np.int64)
    r = np.ascontiguousarray(rows, dtype=np.int64)
    out = np.zeros((r.shape[0], 9), dtype=np.uint32)
    d = None if device is None else np.ascontiguousarray(device, dtype=np.int32)
    _load().oracle_capture_rows(_ptr(a), _ptr(c), None if d is None else _ptr(d), a.shape[0],
                                _ptr(r), r.shape[0], _ptr(out))
    return out
