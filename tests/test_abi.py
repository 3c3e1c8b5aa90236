"""C-ABI checks that need no GPU: the library loads, exports every symbol that
include/lake_linnos.h declares, and host-side argument validation answers without
touching a device."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_asplos_finglertyshar23_b200 import inputs, lake

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared(header="lake_linnos.h", prefix="lake_linnos_"):
    src = open(os.path.join(ROOT, "include", header)).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(" + prefix + r"\w+)\s*\(", src)))


def _all_declared():
    names = []
    for h in sorted(os.listdir(os.path.join(ROOT, "include"))):
        if h.endswith(".h"):
            names += _declared(h, "lake_")
    return sorted(set(names))


def test_header_matches_binding_list():
    assert _declared() == sorted(lake.EXPORTS)
    assert _declared("lake_mlp.h", "lake_mlp_") == sorted(lake.MLP_EXPORTS)
    assert _all_declared() == sorted(lake.EXPORTS + lake.MLP_EXPORTS)


def test_library_exports_every_declared_symbol():
    L = lake.lib()
    for name in _all_declared():
        assert hasattr(L, name), name
    # the binding resolves by the same names
    dl = ctypes.CDLL(lake.LIB_PATH)
    for name in _all_declared():
        getattr(dl, name)


def test_blob_sizes():
    for arch in (0, 1, 2):
        assert lake.blob_floats(arch) == inputs.blob_floats(arch)
    assert lake.blob_floats(0) == 8706
    assert lake.blob_floats(1) == 74498
    assert lake.blob_floats(2) == 140290
    assert lake.blob_floats(7) == 0


def test_strerror_all_codes():
    for s in range(6):
        assert isinstance(lake.strerror(s), str) and lake.strerror(s)
    assert lake.strerror(99) == "unknown status"


def test_host_validation_without_device():
    L = lake.lib()
    # n < 0, bad flags, NULL pointers -> LAKE_ERR_INVAL before any CUDA call
    assert L.lake_linnos_infer(None, 0, -1, 0, None, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_infer(None, 0x8, 10, 0, None, None, None) == lake.LAKE_ERR_INVAL
    # tf32 is a valid precision now: a NULL input is the argument error
    assert L.lake_linnos_infer(None, lake.LAKE_PREC_TF32, 10, 0, None, None, None) == \
        lake.LAKE_ERR_INVAL
    assert L.lake_linnos_infer(None, 0x50, 10, 0, None, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_infer(None, 0, 10, 0, None, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_infer(None, 0, 0, 0, None, None, None) == lake.LAKE_OK  # n == 0
    assert L.lake_linnos_digitize(None, -3, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_digitize(None, 0, None, None) == lake.LAKE_OK
    assert L.lake_linnos_digitize(None, 5, None, None) == lake.LAKE_ERR_INVAL
    blob = np.zeros(10, np.float32)
    assert L.lake_linnos_load_weights(0, 2, blob.ctypes.data, 10, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_load_weights(-1, 2, blob.ctypes.data, 10, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_load_weights(0, 9, blob.ctypes.data, 10, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_unload(5000, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_unload(5, 0) == lake.LAKE_ERR_NOMODEL
    assert L.lake_linnos_multi_group(-1, None, None, 0, None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_workspace_bytes(1 << 24) >= (1 << 24) * 4
    assert L.lake_linnos_host_staging_bytes(1000, lake.LAKE_IN_RAW) >= 36000


def test_nonfinite_blob_rejected():
    L = lake.lib()
    blob = inputs.weights(0, 0).copy()
    blob[5] = np.nan
    assert L.lake_linnos_load_weights(0, 0, blob.ctypes.data, blob.size, 0) == lake.LAKE_ERR_INVAL


def test_launch_counter_resets():
    lake.reset_launch_count()
    assert lake.launch_count() == 0


@pytest.mark.parametrize("path", ["lake.py", "csrc/api.cu", "csrc/mlp_tc.cu", "csrc/mlp_fp32.cu",
                                  "csrc/digitize.cu", "csrc/group.cu"])
def test_product_never_touches_oracle(path):
    src = open(os.path.join(ROOT, "paper_conf_asplos_finglertyshar23_b200", path)).read()
    assert "oracle" not in src.replace("bit-exact with the\n// oracle", "").lower() or \
        "import oracle" not in src
    assert "import oracle" not in src and "liblake_oracle" not in src


def test_auto_thresholds_roundtrip():
    assert [lake.auto_threshold(a) for a in range(3)] == [lake.LAKE_AUTO_TC_MIN_N[a] for a in range(3)]
    lake.set_auto_threshold(1, 777)
    assert lake.auto_threshold(1) == 777
    lake.set_auto_threshold(1, lake.LAKE_AUTO_TC_MIN_N[1])
    with pytest.raises(lake.LakeError):
        lake.set_auto_threshold(5, 1)
    with pytest.raises(lake.LakeError):
        lake.set_auto_threshold(0, -1)


def test_mlp_family_host_validation():
    """NEXT-4 ABI (include/lake_mlp.h): shape / argument errors answer on the host."""
    from paper_conf_asplos_finglertyshar23_b200.inputs import family
    L = lake.lib()
    for name, cfg in family.FAMILY.items():
        assert lake.mlp_blob_floats(cfg["widths"]) == family.blob_floats(cfg["widths"])
    assert lake.mlp_blob_floats([15, 10, 10, 2]) == 15 * 10 + 10 + 10 * 10 + 10 + 10 * 2 + 2
    assert lake.mlp_blob_floats([5, 15, 15, 4]) == 5 * 15 + 15 + 15 * 15 + 15 + 15 * 4 + 4
    for bad in ([3, 1], [0, 4, 2], [3, 65, 2], [3, 4, 4, 4, 4, 2], [3]):
        assert lake.mlp_blob_floats(bad) == 0, bad
    w = np.array([5, 15, 15, 4], np.int32)
    blob = family.weights(w, 0)
    P = w.ctypes.data
    assert L.lake_mlp_load(-1, 3, P, 1, blob.ctypes.data, blob.size, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_load(256, 3, P, 1, blob.ctypes.data, blob.size, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_load(0, 3, P, 2, blob.ctypes.data, blob.size, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_load(0, 3, P, 1, blob.ctypes.data, blob.size - 1, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_load(0, 3, P, 1, None, blob.size, 0) == lake.LAKE_ERR_INVAL
    bad = blob.copy()
    bad[7] = np.inf
    assert L.lake_mlp_load(0, 3, P, 1, bad.ctypes.data, bad.size, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_load(0, 3, P, 1, blob.ctypes.data, blob.size, -1) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_infer(None, -1, 0, None, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_infer(None, 0, 0, None, None, None) == lake.LAKE_OK      # n == 0: no-op
    assert L.lake_mlp_infer(None, 10, 0, None, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_infer(16, 10, 0, 18, None, None) == lake.LAKE_ERR_INVAL  # misaligned
    assert L.lake_mlp_infer(16, 2 ** 31, 0, 32, None, None) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_unload(-1, 0) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_unload(5, 0) == lake.LAKE_ERR_NOMODEL
    assert L.lake_mlp_model_shape(5, 0, None, None, None) == lake.LAKE_ERR_INVAL
    assert lake.mlp_host_staging_bytes(1000, 15, 2) >= 1000 * (15 + 1 + 2) * 4
    assert lake.mlp_host_staging_bytes(-1, 15, 2) == 0 and lake.mlp_host_staging_bytes(10, 65, 2) == 0
    assert L.lake_mlp_infer_host(None, 0, 0, None, None, None, 0, None) == lake.LAKE_OK
    assert L.lake_mlp_infer_host(None, 5, 0, None, None, None, 0, None) == lake.LAKE_ERR_INVAL
    assert L.lake_mlp_infer_host(16, -1, 0, 16, None, None, 0, None) == lake.LAKE_ERR_INVAL


def test_id_width_flags_validated_on_host():
    """bits 8..9 select the model-id element type; 0x300 and unknown bits are rejected."""
    L = lake.lib()
    bad = lake.LAKE_IN_RAW | lake.LAKE_IDS_MASK
    assert L.lake_linnos_infer_multi(16, bad, 10, 16, 16, None, 16, 1 << 20, None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_infer_multi(16, 0x400 | lake.LAKE_IN_RAW, 10, 16, 16, None, 16, 1 << 20,
                                     None) == lake.LAKE_ERR_INVAL
    assert L.lake_linnos_infer_host(16, bad, 10, 0, 16, 16, None, 16, 1 << 30, None) == lake.LAKE_ERR_INVAL
