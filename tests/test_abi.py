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


def _declared():
    src = open(os.path.join(ROOT, "include", "lake_linnos.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lake_linnos_\w+)\s*\(", src)))


def test_header_matches_binding_list():
    assert _declared() == sorted(lake.EXPORTS)


def test_library_exports_every_declared_symbol():
    L = lake.lib()
    for name in _declared():
        assert hasattr(L, name), name
    # the binding resolves by the same names
    dl = ctypes.CDLL(lake.LIB_PATH)
    for name in _declared():
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
    assert L.lake_linnos_infer(None, lake.LAKE_PREC_TF32, 10, 0, None, None, None) == \
        lake.LAKE_ERR_UNSUPPORTED
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
