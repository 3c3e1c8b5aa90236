"""NN-only tensor-core launches (every tile has a single layer, drained alternately by both
epilogue groups; the digitiser gathers before the X-empty wait): single-model batches over
many tiles per CTA pair, digit and raw inputs, and NN-only multi-model grouping with unknown
ids. Expected values only from oracle/ (or, for grouping, the single-model path)."""
import numpy as np
import pytest

import oracle
from gpu_util import run_infer, run_multi, tc_metrics
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake

pytestmark = pytest.mark.gpu
IDS = (400, 401, 402)


@pytest.fixture(scope="module", autouse=True)
def nn_models():
    import torch
    torch.cuda.set_device(0)
    for m in IDS:
        lake.load_weights(m, 0, inputs.weights(0, m), 0)
    yield
    for m in IDS:
        lake.unload(m, 0)


def _check(lg, dec, rlg, rdec):
    met = tc_metrics(lg, dec, rlg, rdec)
    assert met["max_rel"] <= 2e-2 and met["max_disagree_margin"] < 5e-2, met
    assert met["agreement"] >= 0.999, met


@pytest.mark.parametrize("prec", [lake.LAKE_PREC_F16, lake.LAKE_PREC_TF32])
@pytest.mark.parametrize("n", [1, 255, 257, 300_001])
def test_single_model_many_tiles(n, prec):
    raw = inputs.device_trace("azure", n, 91, rerate=3.0)["raw"]
    lg, dec = run_infer(400, raw, lake.LAKE_IN_RAW | prec)
    smp = np.unique(np.concatenate([np.arange(0, n, 37), np.arange(max(0, n - 300), n)]))
    rlg, rdec = oracle.infer_raw(0, inputs.weights(0, 400), raw[smp], nthreads=0)
    _check(lg[smp], dec[smp], rlg, rdec)
    # digit input takes the same pipeline
    import torch
    d = torch.empty((n, 32), dtype=torch.uint8, device="cuda:0")
    x = torch.from_numpy(raw.view(np.int32)).cuda()
    lake.digitize(x, n, d)
    torch.cuda.synchronize()
    lg2, dec2 = run_infer(400, d.cpu().numpy(), lake.LAKE_IN_DIGITS | prec)
    assert np.array_equal(dec2, dec) and np.array_equal(lg2.view(np.uint32), lg.view(np.uint32))


@pytest.mark.parametrize("prec", [lake.LAKE_PREC_F16, lake.LAKE_PREC_BF16, lake.LAKE_PREC_TF32])
def test_multi_nn_equals_per_model(prec):
    raw, mids = inputs.multi_device_trace(400_000, 3, seed_base=4100, rerate=3.0)
    ids = np.array(IDS)[mids].astype(np.int32)
    ids[::997] = 5  # unknown ids in between
    lg, dec, unk = run_multi(raw, ids, lake.LAKE_IN_RAW | prec)
    assert unk == int((ids == 5).sum())
    for m in IDS:
        idx = np.nonzero(ids == m)[0]
        slg, sdec = run_infer(m, raw[idx], lake.LAKE_IN_RAW | prec)
        assert np.array_equal(dec[idx], sdec)
        assert np.array_equal(lg[idx].view(np.uint32), slg.view(np.uint32))
    assert np.all(dec[ids == 5] == 0)


@pytest.mark.parametrize("prec", [lake.LAKE_PREC_F16, lake.LAKE_PREC_TF32, lake.LAKE_PREC_FP32])
def test_many_tiny_model_groups(prec):
    """250 NN+2 models with a skewed I/O count (many groups of 1-3 I/Os): almost every tile
    of every CTA pair switches model (weight-reload protocol at its densest), plus unknown
    ids; grouped results equal the oracle per model."""
    mids = list(range(500, 750))
    blobs = {m: inputs.weights(2, m) for m in mids}
    for m in mids:
        lake.load_weights(m, 2, blobs[m], 0)
    try:
        rng = np.random.default_rng(17)
        p = 1.0 / np.arange(1, len(mids) + 1) ** 1.5
        ids = np.array(mids)[rng.choice(len(mids), size=30000, p=p / p.sum())].astype(np.int32)
        ids[::501] = 9999
        raw = inputs.device_trace("azure", ids.size, 23, rerate=3.0)["raw"]
        lg, dec, unk = run_multi(raw, ids, lake.LAKE_IN_RAW | prec)
        assert unk == int((ids == 9999).sum())
        rlg, rdec = oracle.infer_multi_raw({m: (2, blobs[m]) for m in mids}, raw, ids, nthreads=0)
        ok = ids != 9999
        if prec == lake.LAKE_PREC_FP32:
            assert np.array_equal(dec, rdec)
            assert np.array_equal(lg[ok].view(np.uint32), rlg[ok].view(np.uint32))
        else:
            _check(lg[ok], dec[ok], rlg[ok], rdec[ok])
            assert np.all(dec[~ok] == 0)
    finally:
        for m in mids:
            lake.unload(m, 0)
