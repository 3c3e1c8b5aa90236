"""GPU parity of the NEXT-4 MLP family (include/lake_mlp.h) against oracle.mlp_family.

ReLU models: outputs and classes bit-exact (same operation order, R15).
Sigmoid models: the kernel computes sigmoid on the SFU (ex2.approx / rcp.approx), the oracle
with glibc expf and IEEE division, so outputs are compared within 1e-5 relative (S19 form: |d| / max(|ref|, rms(ref))) and
classes must agree wherever the oracle's top-two margin exceeds 1e-4 (R27/R28).
Inputs come from the seeded generators; expected values only from oracle/."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_asplos_finglertyshar23_b200 import lake
from paper_conf_asplos_finglertyshar23_b200.inputs import family

pytestmark = pytest.mark.gpu
DEV = "cuda:0"

SHAPES = {
    "mllb": (family.FAMILY["mllb"]["widths"], family.ACT_RELU),
    "kml": (family.FAMILY["kml"]["widths"], family.ACT_SIGMOID),
    "w32_sig": ((20, 30, 2), family.ACT_SIGMOID),
    "w64_relu": ((64, 64, 64, 64, 3), family.ACT_RELU),
    "w1_relu": ((1, 1, 2), family.ACT_RELU),
    "even_in": ((16, 8, 5), family.ACT_RELU),
    "c64_sig": ((7, 33, 64), family.ACT_SIGMOID),  # widest output layer, odd hidden width
}


def _run(mid, x, with_out=True):
    n = x.shape[0]
    xd = torch.from_numpy(np.ascontiguousarray(x)).to(DEV)
    cls = torch.full((n,), -7, dtype=torch.int32, device=DEV)
    C = lake.mlp_model_shape(mid, 0)[0][-1]
    out = torch.full((n, C), 12345.0, dtype=torch.float32, device=DEV) if with_out else None
    lake.mlp_infer(xd, n, mid, cls, out)
    torch.cuda.synchronize()
    return (out.cpu().numpy() if with_out else None), cls.cpu().numpy()


def _check(act, o, c, ro, rc):
    if act == family.ACT_RELU:
        assert np.array_equal(o.view(np.uint32), ro.view(np.uint32))
        assert np.array_equal(c, rc)
        return
    ref = ro.astype(np.float64)
    rms = np.sqrt(np.mean(ref ** 2))
    rel = np.abs(o - ref) / np.maximum(np.abs(ref), rms)
    assert rel.max() <= 1e-5, rel.max()
    top2 = np.sort(ref, axis=1)[:, -2:]
    clear = (top2[:, 1] - top2[:, 0]) > 1e-4
    assert np.array_equal(c[clear], rc[clear])
    # where it is not clear, the kernel's class is one of the (near-)maximal outputs
    idx = np.nonzero(~clear)[0]
    assert np.all(ref[idx, c[idx]] >= top2[idx, 1] - 1e-4)


@pytest.fixture(params=["auto", "generic"])
def kernel_path(request):
    """Both kernels: the compile-time-shape one (MLLB / KML shapes) and the generic one."""
    prev = lake.mlp_force_generic(request.param == "generic")
    yield request.param
    lake.mlp_force_generic(prev)


@pytest.mark.parametrize("name", list(SHAPES))
@pytest.mark.parametrize("n", [1, 127, 128, 129, 1000, 4133, 70001])
def test_parity(name, n, kernel_path):
    widths, act = SHAPES[name]
    if kernel_path == "generic" and name not in ("mllb", "kml"):
        pytest.skip("generic is the only kernel for this shape")
    mid = 3
    blob = family.weights(widths, 11)
    lake.mlp_load(mid, widths, act, blob, 0)
    try:
        x = family.features(n, widths[0], 100 + n)
        o, c = _run(mid, x)
        ro, rc = oracle.mlp_family(widths, act, blob, x, nthreads=0)
        _check(act, o, c, ro, rc)
        # classes-only call gives the same classes
        _, c2 = _run(mid, x, with_out=False)
        assert np.array_equal(c2, c)
    finally:
        lake.mlp_unload(mid, 0)


def test_nan_and_saturation_rows(kernel_path):
    widths, act = SHAPES["kml"]
    blob = family.weights(widths, 1)
    lake.mlp_load(0, widths, act, blob, 0)
    x = family.features(300, widths[0], 7)
    x[:50] *= 1e4          # sigmoid saturation
    x[50:60, 2] = np.nan   # NaN -> all outputs NaN -> class 0
    x[60:70] = 0.0
    o, c = _run(0, x)
    ro, rc = oracle.mlp_family(widths, act, blob, x)
    assert np.array_equal(np.isnan(o), np.isnan(ro))
    assert np.all(c[50:60] == 0) and np.all(rc[50:60] == 0)
    fin = ~np.isnan(ro).any(axis=1)
    _check(act, o[fin], c[fin], ro[fin], rc[fin])
    lake.mlp_unload(0, 0)


def test_ties_first_max(kernel_path):
    # output neurons 0 and 1 identical -> exact tie -> class 0 on both sides
    widths = (15, 10, 10, 2)
    blob = family.weights(widths, 4)
    W_out = blob[-(10 * 2 + 2):]
    W_out[10:20] = W_out[0:10]
    W_out[21] = W_out[20]
    lake.mlp_load(1, widths, family.ACT_RELU, blob, 0)
    x = family.features(2000, 15, 3)
    o, c = _run(1, x)
    ro, rc = oracle.mlp_family(widths, family.ACT_RELU, blob, x)
    _check(family.ACT_RELU, o, c, ro, rc)
    assert np.all(c == 0)
    lake.mlp_unload(1, 0)


def test_determinism_and_batch_independence():
    widths, act = SHAPES["kml"]
    blob = family.weights(widths, 5)
    lake.mlp_load(2, widths, act, blob, 0)
    x = family.features(50000, widths[0], 9)
    o1, c1 = _run(2, x)
    o2, c2 = _run(2, x)
    assert np.array_equal(o1.view(np.uint32), o2.view(np.uint32)) and np.array_equal(c1, c2)
    os_, cs = _run(2, x[12345:12345 + 77].copy())
    assert np.array_equal(os_.view(np.uint32), o1[12345:12345 + 77].view(np.uint32))
    lake.mlp_unload(2, 0)


def test_errors_and_shape():
    widths, act = SHAPES["mllb"]
    blob = family.weights(widths, 0)
    lake.mlp_load(9, widths, act, blob, 0)
    assert lake.mlp_model_shape(9, 0) == (tuple(widths), act)
    lake.mlp_unload(9, 0)
    x = torch.zeros((4, widths[0]), device=DEV)
    cls = torch.zeros(4, dtype=torch.int32, device=DEV)
    with pytest.raises(lake.LakeError) as e:
        lake.mlp_infer(x, 4, 9, cls)
    assert e.value.status == lake.LAKE_ERR_NOMODEL
    with pytest.raises(lake.LakeError):
        lake.mlp_model_shape(9, 0)


@pytest.mark.parametrize("name", ["mllb", "kml"])
def test_full_size_sampled(name, kernel_path):
    """The bench's configuration (2^24 rows, the launch bench.py times), checked on a
    sampled subset of rows the oracle computes one by one."""
    widths, act = SHAPES[name]
    n = 1 << 24
    blob = family.weights(widths, 0)
    lake.mlp_load(4, widths, act, blob, 0)
    x = family.features(n, widths[0], 2024)
    o, c = _run(4, x)
    rows = np.unique(np.concatenate([np.arange(0, n, 4099), np.arange(n - 300, n)]))
    ro, rc = oracle.mlp_family(widths, act, blob, x[rows], nthreads=0)
    _check(act, o[rows], c[rows], ro, rc)
    lake.mlp_unload(4, 0)


@pytest.mark.parametrize("name", ["mllb", "kml"])
def test_unaligned_input_rows(name, kernel_path):
    """x not 16-byte aligned: the kernel falls back from the bulk (TMA) row copy to 4-byte
    cp.async copies; results are the same."""
    widths, act = SHAPES[name]
    blob = family.weights(widths, 6)
    lake.mlp_load(5, widths, act, blob, 0)
    n = 50000 + 3
    x = family.features(n, widths[0], 77)
    buf = torch.zeros(n * widths[0] + 1, dtype=torch.float32, device=DEV)
    buf[1:] = torch.from_numpy(x.ravel()).to(DEV)
    xd = buf[1:]
    assert xd.data_ptr() % 16 != 0
    cls = torch.full((n,), -7, dtype=torch.int32, device=DEV)
    out = torch.full((n, widths[-1]), 12345.0, dtype=torch.float32, device=DEV)
    lake.mlp_infer(xd, n, 5, cls, out)
    torch.cuda.synchronize()
    ro, rc = oracle.mlp_family(widths, act, blob, x, nthreads=0)
    _check(act, out.cpu().numpy(), cls.cpu().numpy(), ro, rc)
    lake.mlp_unload(5, 0)


@pytest.mark.parametrize("pinned", [True, False])
@pytest.mark.parametrize("n", [1, 100, 5000])
def test_infer_host_equals_device(pinned, n):
    """lake_mlp_infer_host: zero-copy (pinned, mapped) and staged (pageable) host buffers
    give the device path's results bit for bit."""
    widths, act = SHAPES["kml"]
    blob = family.weights(widths, 8)
    lake.mlp_load(6, widths, act, blob, 0)
    x = family.features(n, widths[0], 31)
    o, c = _run(6, x)
    C = widths[-1]
    if pinned:
        hx = torch.from_numpy(x).pin_memory()
        hc = torch.full((n,), -7, dtype=torch.int32).pin_memory()
        ho = torch.full((n, C), 12345.0, dtype=torch.float32).pin_memory()
        lake.mlp_infer_host(hx, n, 6, hc, ho)
        hc, ho = hc.numpy(), ho.numpy()
    else:
        hx = np.ascontiguousarray(x)
        hc = np.full(n, -7, np.int32)
        ho = np.full((n, C), 12345.0, np.float32)
        sb = lake.mlp_host_staging_bytes(n, widths[0], C)
        stg = torch.empty(sb, dtype=torch.uint8, device=DEV)
        lake.mlp_infer_host(hx, n, 6, hc, ho, stg, sb)
    assert np.array_equal(hc, c)
    assert np.array_equal(ho.view(np.uint32), o.view(np.uint32))
    lake.mlp_unload(6, 0)
