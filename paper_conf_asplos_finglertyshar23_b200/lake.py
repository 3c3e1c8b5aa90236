"""Thin Python binding of the C ABI in include/lake_linnos.h (argument marshalling only).

Every function has the C name without the ``lake_linnos_`` prefix and the same argument
order; device buffers are torch CUDA tensors (or raw integer pointers), streams default to
torch's current stream. All arithmetic runs in liblake_linnos.so's CUDA kernels; there is
no CPU fallback: if the library is missing or fails to load, every call raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liblake_linnos.so")
# development only: scripts/trace_tc.py points this at the timeline-trace build
LIB_PATH = os.environ.get("LAKE_LINNOS_LIB", LIB_PATH)

# enums / flags (mirrors include/lake_linnos.h)
LAKE_OK, LAKE_ERR_INVAL, LAKE_ERR_NOMODEL, LAKE_ERR_CUDA, LAKE_ERR_NOMEM, LAKE_ERR_UNSUPPORTED = range(6)
LAKE_ARCH_NN, LAKE_ARCH_NN1, LAKE_ARCH_NN2 = 0, 1, 2
LAKE_IN_DIGITS, LAKE_IN_RAW = 0x00, 0x01
LAKE_PREC_FP32, LAKE_PREC_F16, LAKE_PREC_BF16, LAKE_PREC_TF32, LAKE_PREC_AUTO = (
    0x00, 0x10, 0x20, 0x30, 0x70)
LAKE_IDS_I32, LAKE_IDS_U16, LAKE_IDS_U8, LAKE_IDS_MASK = 0x000, 0x100, 0x200, 0x300
LAKE_MAX_MODELS = 1024
LAKE_SERVER_MAX_BATCH = 64
LAKE_AUTO_TC_MIN_N = {0: 8192, 1: 1, 2: 1}  # defaults (include/lake_linnos.h)

PREC_FLAGS = {"fp32": LAKE_PREC_FP32, "f16": LAKE_PREC_F16, "bf16": LAKE_PREC_BF16,
              "tf32": LAKE_PREC_TF32, "auto": LAKE_PREC_AUTO}

# every symbol include/lake_linnos.h declares (checked by tests/test_abi.py)
EXPORTS = (
    "lake_linnos_blob_floats", "lake_linnos_load_weights", "lake_linnos_unload",
    "lake_linnos_model_arch", "lake_linnos_digitize", "lake_linnos_infer",
    "lake_linnos_workspace_bytes", "lake_linnos_infer_multi", "lake_linnos_multi_group",
    "lake_linnos_multi_grouped", "lake_linnos_multi_status", "lake_linnos_host_staging_bytes",
    "lake_linnos_infer_host", "lake_linnos_launch_count", "lake_linnos_reset_launch_count",
    "lake_linnos_profile_enable", "lake_linnos_profile_read", "lake_linnos_strerror",
    "lake_linnos_capture_workspace_bytes", "lake_linnos_capture",
    "lake_linnos_auto_threshold", "lake_linnos_set_auto_threshold",
    "lake_linnos_server_start", "lake_linnos_server_infer", "lake_linnos_server_stop",
)
# every symbol include/lake_mlp.h declares (NEXT-4 MLP family)
MLP_EXPORTS = (
    "lake_mlp_blob_floats", "lake_mlp_load", "lake_mlp_unload", "lake_mlp_infer",
    "lake_mlp_model_shape", "lake_mlp_force_generic", "lake_mlp_host_staging_bytes",
    "lake_mlp_infer_host",
)
LAKE_ACT_RELU, LAKE_ACT_SIGMOID = 0, 1
LAKE_MLP_MAX_LAYERS, LAKE_MLP_MAX_WIDTH, LAKE_MLP_MAX_MODELS = 4, 64, 256


class LakeError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: {strerror(status)} ({status})")
        self.status = status


_lib = None


def lib():
    """Load liblake_linnos.so (built in-tree by `make`). Raises if it is missing."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run `make` (or __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        P, I32, I64, U32, SZ = (ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64,
                                ctypes.c_uint32, ctypes.c_size_t)
        sig = {
            "lake_linnos_blob_floats": (SZ, [I32]),
            "lake_linnos_load_weights": (ctypes.c_int, [I32, I32, P, SZ, I32]),
            "lake_linnos_unload": (ctypes.c_int, [I32, I32]),
            "lake_linnos_model_arch": (ctypes.c_int, [I32, I32, P]),
            "lake_linnos_digitize": (ctypes.c_int, [P, I64, P, P]),
            "lake_linnos_infer": (ctypes.c_int, [P, U32, I64, I32, P, P, P]),
            "lake_linnos_workspace_bytes": (SZ, [I64]),
            "lake_linnos_infer_multi": (ctypes.c_int, [P, U32, I64, P, P, P, P, SZ, P]),
            "lake_linnos_multi_group": (ctypes.c_int, [I64, P, P, SZ, P]),
            "lake_linnos_multi_grouped": (ctypes.c_int, [P, U32, I64, P, P, P, SZ, P]),
            "lake_linnos_multi_status": (ctypes.c_int, [P, SZ, P, P]),
            "lake_linnos_host_staging_bytes": (SZ, [I64, U32]),
            "lake_linnos_infer_host": (ctypes.c_int, [P, U32, I64, I32, P, P, P, P, SZ, P]),
            "lake_linnos_launch_count": (ctypes.c_uint64, []),
            "lake_linnos_reset_launch_count": (None, []),
            "lake_linnos_profile_enable": (ctypes.c_int, [ctypes.c_int]),
            "lake_linnos_profile_read": (ctypes.c_int, [P, P]),
            "lake_linnos_strerror": (ctypes.c_char_p, [ctypes.c_int]),
            "lake_linnos_capture_workspace_bytes": (SZ, [I64]),
            "lake_linnos_capture": (ctypes.c_int, [P, P, P, I64, P, P, SZ, P]),
            "lake_linnos_auto_threshold": (ctypes.c_int, [I32, P]),
            "lake_linnos_set_auto_threshold": (ctypes.c_int, [I32, I64]),
            "lake_linnos_server_start": (ctypes.c_int, [I32, P]),
            "lake_linnos_server_infer": (ctypes.c_int, [P, P, I32, P, P]),
            "lake_linnos_server_stop": (ctypes.c_int, [P]),
            "lake_mlp_blob_floats": (SZ, [I32, P]),
            "lake_mlp_load": (ctypes.c_int, [I32, I32, P, I32, P, SZ, I32]),
            "lake_mlp_unload": (ctypes.c_int, [I32, I32]),
            "lake_mlp_infer": (ctypes.c_int, [P, I64, I32, P, P, P]),
            "lake_mlp_model_shape": (ctypes.c_int, [I32, I32, P, P, P]),
            "lake_mlp_force_generic": (ctypes.c_int, [I32]),
            "lake_mlp_host_staging_bytes": (SZ, [I64, I32, I32]),
            "lake_mlp_infer_host": (ctypes.c_int, [P, I64, I32, P, P, P, SZ, P]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def strerror(status: int) -> str:
    return lib().lake_linnos_strerror(status).decode()


def _ptr(x):
    """Device/host pointer of a torch tensor, numpy array, int, or None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return x.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _check(rc: int, what: str) -> None:
    if rc != LAKE_OK:
        raise LakeError(rc, what)


def blob_floats(arch: int) -> int:
    return int(lib().lake_linnos_blob_floats(arch))


def load_weights(model_id: int, arch: int, blob: np.ndarray, device: int) -> None:
    blob = np.ascontiguousarray(blob, dtype=np.float32)
    _check(lib().lake_linnos_load_weights(model_id, arch, blob.ctypes.data, blob.size, device),
           "load_weights")


def unload(model_id: int, device: int) -> None:
    _check(lib().lake_linnos_unload(model_id, device), "unload")


def model_arch(model_id: int, device: int) -> int:
    out = ctypes.c_int32(-1)
    _check(lib().lake_linnos_model_arch(model_id, device, ctypes.byref(out)), "model_arch")
    return out.value


def digitize(raw, n: int, digits, stream=None) -> None:
    _check(lib().lake_linnos_digitize(_ptr(raw), n, _ptr(digits), _stream(stream)), "digitize")


def infer(inp, flags: int, n: int, model_id: int, decisions, logits=None, stream=None) -> None:
    _check(lib().lake_linnos_infer(_ptr(inp), flags, n, model_id, _ptr(decisions), _ptr(logits),
                                   _stream(stream)), "infer")


def workspace_bytes(n: int) -> int:
    return int(lib().lake_linnos_workspace_bytes(n))


def infer_multi(inp, flags: int, n: int, model_ids, decisions, logits, workspace, ws_bytes: int,
                stream=None) -> None:
    _check(lib().lake_linnos_infer_multi(_ptr(inp), flags, n, _ptr(model_ids), _ptr(decisions),
                                         _ptr(logits), _ptr(workspace), ws_bytes,
                                         _stream(stream)), "infer_multi")


def multi_group(n: int, model_ids, workspace, ws_bytes: int, stream=None) -> None:
    _check(lib().lake_linnos_multi_group(n, _ptr(model_ids), _ptr(workspace), ws_bytes,
                                         _stream(stream)), "multi_group")


def multi_grouped(inp, flags: int, n: int, decisions, logits, workspace, ws_bytes: int,
                  stream=None) -> None:
    _check(lib().lake_linnos_multi_grouped(_ptr(inp), flags, n, _ptr(decisions), _ptr(logits),
                                           _ptr(workspace), ws_bytes, _stream(stream)),
           "multi_grouped")


def multi_status(workspace, ws_bytes: int, stream=None) -> int:
    out = ctypes.c_int64(0)
    _check(lib().lake_linnos_multi_status(_ptr(workspace), ws_bytes, ctypes.addressof(out),
                                          _stream(stream)), "multi_status")
    return out.value


def host_staging_bytes(n: int, flags: int) -> int:
    return int(lib().lake_linnos_host_staging_bytes(n, flags))


def infer_host(h_in, flags: int, n: int, model_id: int, h_model_ids, h_decisions, h_logits,
               d_staging, staging_bytes: int, stream=None) -> None:
    _check(lib().lake_linnos_infer_host(_ptr(h_in), flags, n, model_id, _ptr(h_model_ids),
                                        _ptr(h_decisions), _ptr(h_logits), _ptr(d_staging),
                                        staging_bytes, _stream(stream)), "infer_host")


def launch_count() -> int:
    return int(lib().lake_linnos_launch_count())


def reset_launch_count() -> None:
    lib().lake_linnos_reset_launch_count()


def profile_enable(enable: bool) -> None:
    _check(lib().lake_linnos_profile_enable(1 if enable else 0), "profile_enable")


def profile_read():
    ms = ctypes.c_double(0.0)
    n = ctypes.c_int64(0)
    _check(lib().lake_linnos_profile_read(ctypes.addressof(ms), ctypes.addressof(n)),
           "profile_read")
    return ms.value, n.value


def capture_workspace_bytes(n: int) -> int:
    return int(lib().lake_linnos_capture_workspace_bytes(n))


def capture(arrival_ns, complete_ns, device, n: int, raw_out, workspace, ws_bytes: int,
            stream=None) -> None:
    _check(lib().lake_linnos_capture(_ptr(arrival_ns), _ptr(complete_ns), _ptr(device), n,
                                     _ptr(raw_out), _ptr(workspace), ws_bytes, _stream(stream)),
           "capture")


def auto_threshold(arch: int) -> int:
    out = ctypes.c_int64(0)
    _check(lib().lake_linnos_auto_threshold(arch, ctypes.addressof(out)), "auto_threshold")
    return out.value


def set_auto_threshold(arch: int, n_min: int) -> None:
    _check(lib().lake_linnos_set_auto_threshold(arch, n_min), "set_auto_threshold")


class Server:
    """Persistent resident-weights server (lake_linnos_server_*): host buffers in and out."""

    def __init__(self, model_id: int):
        self._h = ctypes.c_void_p(0)
        _check(lib().lake_linnos_server_start(model_id, ctypes.byref(self._h)), "server_start")

    def infer(self, h_raw, n: int, h_decisions, h_logits=None) -> None:
        _check(lib().lake_linnos_server_infer(self._h, _ptr(h_raw), n, _ptr(h_decisions),
                                              _ptr(h_logits)), "server_infer")

    def stop(self) -> None:
        if self._h:
            _check(lib().lake_linnos_server_stop(self._h), "server_stop")
            self._h = ctypes.c_void_p(0)

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.stop()


# ---------------------------------------------------------------- NEXT-4 MLP family
def mlp_blob_floats(widths) -> int:
    w = np.ascontiguousarray(widths, dtype=np.int32)
    return int(lib().lake_mlp_blob_floats(len(w) - 1, w.ctypes.data))


def mlp_load(model_id: int, widths, act: int, blob: np.ndarray, device: int) -> None:
    w = np.ascontiguousarray(widths, dtype=np.int32)
    blob = np.ascontiguousarray(blob, dtype=np.float32)
    _check(lib().lake_mlp_load(model_id, len(w) - 1, w.ctypes.data, act, blob.ctypes.data,
                               blob.size, device), "mlp_load")


def mlp_unload(model_id: int, device: int) -> None:
    _check(lib().lake_mlp_unload(model_id, device), "mlp_unload")


def mlp_infer(x, n: int, model_id: int, classes, out=None, stream=None) -> None:
    _check(lib().lake_mlp_infer(_ptr(x), n, model_id, _ptr(classes), _ptr(out),
                                _stream(stream)), "mlp_infer")


def mlp_model_shape(model_id: int, device: int):
    nl = ctypes.c_int32(0)
    act = ctypes.c_int32(-1)
    w = np.zeros(LAKE_MLP_MAX_LAYERS + 1, dtype=np.int32)
    _check(lib().lake_mlp_model_shape(model_id, device, ctypes.byref(nl), w.ctypes.data,
                                      ctypes.byref(act)), "mlp_model_shape")
    return tuple(int(v) for v in w[: nl.value + 1]), act.value


def mlp_force_generic(enable: bool) -> bool:
    """Route every MLP-family model through the generic kernel; returns the previous value."""
    return bool(lib().lake_mlp_force_generic(1 if enable else 0))


def mlp_host_staging_bytes(n: int, width_in: int, classes: int) -> int:
    return int(lib().lake_mlp_host_staging_bytes(n, width_in, classes))


def mlp_infer_host(h_x, n: int, model_id: int, h_classes, h_out=None, d_staging=None,
                   staging_bytes: int = 0, stream=None) -> None:
    _check(lib().lake_mlp_infer_host(_ptr(h_x), n, model_id, _ptr(h_classes), _ptr(h_out),
                                     _ptr(d_staging), staging_bytes, _stream(stream)),
           "mlp_infer_host")
