"""Pins for the oracle's NEXT-4 MLP family (oracle.mlp_family; readings R25-R28).

Each test checks the oracle against something other than itself:
* hand-worked examples (tests/golden/family_examples.txt): sigma(0) = 0.5, saturation,
  first-max ties, NaN -> class 0;
* randomised integer ReLU MLPs with C = 4 classes against exact int64 arithmetic, with
  forced output ties (first max wins);
* sigmoid: the reflection sigma(-z) = 1 - sigma(z) turned into an output identity, and a
  numpy float64 chain (library special case) within the binary32 error bound;
* C = 2 ReLU networks equal the LinnOS oracle (oracle.mlp, pinned separately) bit for bit;
* batch independence.
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden
from paper_conf_asplos_finglertyshar23_b200.inputs import family

GOLDEN_W = np.array([1, -1, 0, 0, 0, 200, 2, 0, 0, 3, 2, -1, 0, -1, 0.5], np.float32)


@pytest.mark.parametrize("row", read_golden("family_examples.txt"), ids=lambda r: r[0])
def test_hand_worked(row):
    name, act, x, out, cls = row
    x = np.array([float(v) for v in x.split()], np.float32)[None, :]
    o, c = oracle.mlp_family([2, 2, 3], int(act), GOLDEN_W, x)
    exp = np.array([float(v) for v in out.split()], np.float32)
    assert np.array_equal(o[0], exp, equal_nan=True), (o[0], exp)
    assert int(c[0]) == int(cls)


def _int_ref(widths, Ws, bs, x):
    h = x.astype(np.int64)
    for l, (W, b) in enumerate(zip(Ws, bs)):
        z = h @ W.astype(np.int64).T + b.astype(np.int64)
        h = np.maximum(z, 0) if l + 1 < len(Ws) else z
    return h


@pytest.mark.parametrize("widths", [(3, 4, 4), (5, 7, 6, 4), (15, 10, 10, 2), (2, 3, 3, 3, 5)])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_integer_relu_exact(widths, seed):
    rng = np.random.default_rng(seed)
    Ws = [rng.integers(-3, 4, size=(widths[l + 1], widths[l])) for l in range(len(widths) - 1)]
    bs = [rng.integers(-4, 5, size=widths[l + 1]) for l in range(len(widths) - 1)]
    # force exact ties on half the rows: duplicate output neuron 0 into neuron 1
    Ws_t = [w.copy() for w in Ws]
    bs_t = [b.copy() for b in bs]
    Ws_t[-1][1] = Ws_t[-1][0]
    bs_t[-1][1] = bs_t[-1][0]
    x = rng.integers(-6, 7, size=(64, widths[0]))
    for W_, b_ in ((Ws, bs), (Ws_t, bs_t)):
        blob = np.concatenate([np.concatenate([w.ravel(), b]) for w, b in zip(W_, b_)]).astype(np.float32)
        o, c = oracle.mlp_family(widths, oracle.ACT_RELU, blob, x.astype(np.float32))
        ref = _int_ref(widths, W_, b_, x)
        assert np.abs(ref).max() < 2 ** 24
        assert np.array_equal(o.astype(np.int64), ref)
        first_max = np.array([list(r).index(max(r)) for r in ref.tolist()])
        assert np.array_equal(c, first_max)


def _blob(Ws, bs):
    return np.concatenate([np.concatenate([w.ravel(), b]) for w, b in zip(Ws, bs)]).astype(np.float32)


def _split(widths, blob):
    Ws, bs, p = [], [], 0
    for l in range(len(widths) - 1):
        k, n = widths[l], widths[l + 1]
        Ws.append(blob[p:p + n * k].reshape(n, k).copy())
        p += n * k
        bs.append(blob[p:p + n].copy())
        p += n
    return Ws, bs


def test_sigmoid_reflection():
    """sigma(-z) = 1 - sigma(z): negating the hidden layer's W, b and folding the
    complement into the output layer (W' = -W, b' = b + W.1) leaves the outputs unchanged
    up to rounding. A sign error in the exponent or a dropped '1 +' breaks it."""
    widths = (5, 15, 4)
    blob = family.weights(widths, 3)
    (W0, W1), (b0, b1) = _split(widths, blob)
    x = family.features(512, 5, 11)
    o, _ = oracle.mlp_family(widths, oracle.ACT_SIGMOID, blob, x)
    W1n = -W1
    b1n = (b1.astype(np.float64) + W1.astype(np.float64).sum(axis=1)).astype(np.float32)
    o2, _ = oracle.mlp_family(widths, oracle.ACT_SIGMOID, _blob([-W0, W1n], [-b0, b1n]), x)
    assert np.allclose(o, o2, rtol=0, atol=2e-6)


def test_sigmoid_range_and_monotone():
    # one hidden unit with weight 1 feeding one output with weight 1: out0 = sigma(x)
    blob = np.array([1, 0, 1, 0, 0, 0], np.float32)  # W0[1][1], b0[1], Wout[2][1], bout[2]
    xs = np.linspace(-30, 30, 601, dtype=np.float32)[:, None]
    o, c = oracle.mlp_family([1, 1, 2], oracle.ACT_SIGMOID, blob, xs)
    s = o[:, 0]
    assert np.all(np.diff(s) >= 0) and s.min() >= 0 and s.max() <= 1
    assert s[300] == 0.5                       # sigma(0)
    assert np.all(c == (s < 0).astype(np.int32))  # out1 = 0: class 1 only if sigma < 0 (never)


@pytest.mark.parametrize("name", ["mllb", "kml"])
def test_float64_chain(name):
    """Library special case: the same network in numpy float64 (matmul + exp) agrees to
    within binary32 rounding (a few ulp per layer)."""
    cfg = family.FAMILY[name]
    widths = cfg["widths"]
    blob = family.weights(widths, 0)
    x = family.features(2048, widths[0], 5)
    o, c = oracle.mlp_family(widths, cfg["act"], blob, x)
    Ws, bs = _split(widths, blob)
    h = x.astype(np.float64)
    for l, (W, b) in enumerate(zip(Ws, bs)):
        z = h @ W.astype(np.float64).T + b
        if l + 1 < len(Ws):
            h = np.maximum(z, 0) if cfg["act"] == 0 else 1.0 / (1.0 + np.exp(-z))
        else:
            h = z
    scale = np.maximum(np.abs(h), np.sqrt(np.mean(h ** 2)))
    assert np.max(np.abs(o - h) / scale) < 1e-5
    top2 = np.sort(h, axis=1)[:, -2:]
    clear = (top2[:, 1] - top2[:, 0]) > 1e-4
    assert np.array_equal(c[clear], np.argmax(h, axis=1)[clear])


def test_two_class_relu_equals_linnos_oracle():
    from paper_conf_asplos_finglertyshar23_b200 import inputs
    blob = inputs.weights(0, 1)
    x = np.random.default_rng(4).integers(0, 10, size=(300, 31)).astype(np.float32)
    lg, dec = oracle.mlp([31, 256, 2], blob, x)
    o, c = oracle.mlp_family([31, 256, 2], oracle.ACT_RELU, blob, x)
    assert np.array_equal(o.view(np.uint32), lg.view(np.uint32))
    assert np.array_equal(c, dec.astype(np.int32))


@pytest.mark.parametrize("name", ["mllb", "kml"])
def test_batch_and_thread_independence(name):
    cfg = family.FAMILY[name]
    widths = cfg["widths"]
    blob = family.weights(widths, 2)
    x = family.features(1000, widths[0], 8)
    o, c = oracle.mlp_family(widths, cfg["act"], blob, x, nthreads=4)
    o1, c1 = oracle.mlp_family(widths, cfg["act"], blob, x[517:518], nthreads=1)
    assert np.array_equal(o[517:518].view(np.uint32), o1.view(np.uint32))
    assert c[517] == c1[0]
    o2, c2 = oracle.mlp_family(widths, cfg["act"], blob, x[::-1].copy(), nthreads=1)
    assert np.array_equal(o[::-1].view(np.uint32), o2.view(np.uint32))


def test_rejects_bad_shapes():
    with pytest.raises(ValueError):
        oracle.mlp_family([3, 4, 1], 0, np.zeros(4 * 3 + 4 + 4 + 1, np.float32), np.zeros((1, 3)))
    with pytest.raises(ValueError):
        oracle.mlp_family([3, 4, 2], 7, np.zeros(4 * 3 + 4 + 8 + 2, np.float32), np.zeros((1, 3)))
