"""Pins for the oracle's MLP + argmax (readings R11-R15).

Each test checks the oracle against something other than itself:
* hand-worked tiny integer MLP (tests/golden/tiny_mlp_examples.txt),
* randomised integer MLPs against exact int64 arithmetic (all intermediates < 2^24,
  so binary32 is exact and must equal the integers bit for bit),
* hand-derived IEEE-754 examples fixing the R15 operation order
  (tests/golden/fp32_order_examples.txt),
* invariants: ReLU zeroing, argmax symmetry, batch independence, thread independence,
  hidden-unit permutation,
* the full-size networks against a numpy float64 GEMM chain (library special case).
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden
from paper_conf_asplos_finglertyshar23_b200 import inputs

ARCHS = [0, 1, 2]


def _digits_of(name):
    for n, rec, dig, s in read_golden("digitize_examples.txt"):
        if n == name:
            return np.array([int(v) for v in dig.split()], dtype=np.float32)
    raise KeyError(name)


def _tiny_blob(swap=False):
    W0 = np.zeros((2, 31), np.float32)
    W0[0, :] = 1
    W0[1, :] = np.where(np.arange(31) % 2 == 0, 1, -1)
    b0 = np.array([-10, 0], np.float32)
    Wout = np.eye(2, dtype=np.float32)
    if swap:
        Wout = Wout[::-1].copy()
    bout = np.zeros(2, np.float32)
    return np.concatenate([W0.ravel(), b0, Wout.ravel(), bout])


@pytest.mark.parametrize("row", read_golden("tiny_mlp_examples.txt"), ids=lambda r: r[0])
def test_tiny_integer_mlp_hand_worked(row):
    name, logits, dec, slogits, sdec = row
    x = _digits_of(name)[None, :]
    lg, d = oracle.mlp([31, 2, 2], _tiny_blob(), x)
    assert lg[0].tolist() == [float(v) for v in logits.split()]
    assert int(d[0]) == int(dec)
    lg, d = oracle.mlp([31, 2, 2], _tiny_blob(swap=True), x)
    assert lg[0].tolist() == [float(v) for v in slogits.split()]
    assert int(d[0]) == int(sdec)


def _int_mlp_int64(widths, Ws, bs, x):
    h = x.astype(np.int64)
    for l, (W, b) in enumerate(zip(Ws, bs)):
        z = h @ W.astype(np.int64).T + b.astype(np.int64)
        h = np.maximum(z, 0) if l + 1 < len(Ws) else z
    return h


@pytest.mark.parametrize("widths", [(31, 2, 2), (31, 4, 4, 2), (31, 8, 2)])
def test_random_integer_mlp_exact(widths):
    raw = inputs.edge_raw(100_000, seed=3)
    x = oracle.digitize(raw).astype(np.float32)
    for seed in range(100):  # first seed whose network is not degenerate (dead hidden units)
        rng = np.random.default_rng(seed)
        Ws = [rng.integers(-3, 4, size=(widths[i + 1], widths[i])) for i in range(len(widths) - 1)]
        bs = [rng.integers(-3, 4, size=widths[i + 1]) for i in range(len(widths) - 1)]
        pre = _int_mlp_int64(widths, Ws, bs, x)
        if np.mean(pre[:, 1] - pre[:, 0] != np.median(pre[:, 1] - pre[:, 0])) > 0.3:
            break
    # centre the class-1 output bias on the integer median margin so both classes occur
    bs[-1][1] -= int(np.median(pre[:, 1] - pre[:, 0]))
    blob = np.concatenate([np.concatenate([W.ravel(), b]) for W, b in zip(Ws, bs)]).astype(np.float32)
    lg, d = oracle.mlp(widths, blob, x, nthreads=0)
    ref = _int_mlp_int64(widths, Ws, bs, x)
    assert np.abs(ref).max() < 2**24
    assert np.array_equal(lg.astype(np.int64), ref)
    assert np.array_equal(d, (ref[:, 1] > ref[:, 0]).astype(np.uint8))
    assert d.min() == 0 and d.max() == 1  # both classes exercised


@pytest.mark.parametrize("row", read_golden("fp32_order_examples.txt"), ids=lambda r: r[0])
def test_fp32_operation_order(row):
    name, widths, x, w, b0, expect, other = row
    widths = [int(v) for v in widths.split()]
    nin = widths[0]
    W = np.zeros((2, nin), np.float32)
    W[0] = [float(v) for v in w.split()]
    b = np.array([float(b0), 0.0], np.float32)
    blob = np.concatenate([W.ravel(), b])
    lg, _ = oracle.mlp(widths, blob, np.array([[float(v) for v in x.split()]], np.float32))
    assert lg[0, 0] == np.float32(float(expect)), (name, lg[0, 0])
    assert lg[0, 0] != np.float32(float(other))


def test_nan_and_tie_give_fast():
    # R14: ties and NaN -> decision 0; ReLU maps NaN to +0 (z > 0 is false).
    inf = np.array([[np.inf]], np.float32)
    blob = np.array([0.0, 0.0, 0.0, 0.0], np.float32)  # widths 1 -> 2: W=[[0],[0]], b=0
    lg, d = oracle.mlp([1, 2], blob, inf)
    assert np.isnan(lg).all() and d[0] == 0
    blob = np.array([0.0, 0.0, 1.0, 1.0, 0.0, 0.0], np.float32)  # 1 -> 1 (relu) -> 2
    lg, d = oracle.mlp([1, 1, 2], blob, inf)
    assert lg[0].tolist() == [0.0, 0.0] and d[0] == 0
    lg, d = oracle.mlp([1, 2], np.array([1.0, 1.0, 0.5, 0.5], np.float32),
                       np.array([[2.0]], np.float32))
    assert lg[0, 0] == lg[0, 1] and d[0] == 0


def _slices(arch, blob):
    w = inputs.ARCH_WIDTHS[arch]
    out, p = [], 0
    for l in range(len(w) - 1):
        W = blob[p:p + w[l + 1] * w[l]].reshape(w[l + 1], w[l]); p += w[l + 1] * w[l]
        b = blob[p:p + w[l + 1]]; p += w[l + 1]
        out.append((W, b))
    return out


def _f64_chain(arch, blob, x):
    h = x.astype(np.float64)
    layers = _slices(arch, blob)
    for l, (W, b) in enumerate(layers):
        h = h @ W.astype(np.float64).T + b.astype(np.float64)
        if l + 1 < len(layers):
            h = np.maximum(h, 0.0)
    return h


@pytest.mark.parametrize("arch", ARCHS)
def test_full_size_vs_float64_gemm_chain(arch):
    raw = inputs.device_trace("azure", 3000, seed=21, rerate=3.0)["raw"]
    raw = np.concatenate([raw, inputs.edge_raw(1000, seed=22)])
    blob = inputs.weights(arch, 5)
    lg, d = oracle.infer_raw(arch, blob, raw, nthreads=0)
    ref = _f64_chain(arch, blob, oracle.digitize(raw).astype(np.float64))
    rms = np.sqrt((ref ** 2).mean())
    err = np.abs(lg - ref) / np.maximum(np.abs(ref), rms)
    assert err.max() < 2e-5, err.max()
    margin = ref[:, 1] - ref[:, 0]
    agree = d == (margin > 0)
    assert np.all(agree | (np.abs(margin) < 1e-4 * rms))


@pytest.mark.parametrize("arch", ARCHS)
def test_relu_zeroing(arch):
    blob = inputs.weights(arch, 1).copy()
    layers = _slices(arch, blob)
    layers[0][1][:] = -1e4          # b0 -> every first-layer unit is negative
    x = oracle.digitize(inputs.edge_raw(500, seed=4)).astype(np.float32)
    lg, _ = oracle.mlp(inputs.ARCH_WIDTHS[arch], blob, x)
    if arch == 0:
        # hidden all zero -> logits are exactly b_out
        assert np.array_equal(lg, np.broadcast_to(layers[-1][1], lg.shape))
    else:
        # closed form: every row equals W_out . ReLU(... ReLU(b1) ...) + b_out
        assert np.all(lg == lg[0])
        h = np.zeros(256)
        for W, b in layers[1:-1]:
            h = np.maximum(W.astype(np.float64) @ h + b, 0.0)
        ref = layers[-1][0].astype(np.float64) @ h + layers[-1][1]
        assert np.allclose(lg[0], ref, rtol=1e-5, atol=1e-6)


@pytest.mark.parametrize("arch", ARCHS)
def test_argmax_symmetry(arch):
    blob = inputs.weights(arch, 2)
    sw = blob.copy()
    Wout, bout = _slices(arch, sw)[-1]
    Wout[:] = Wout[::-1].copy()
    bout[:] = bout[::-1].copy()
    raw = inputs.device_trace("cosmos", 2000, seed=5)["raw"]
    lg, d = oracle.infer_raw(arch, blob, raw)
    lg2, d2 = oracle.infer_raw(arch, sw, raw)
    assert np.array_equal(lg2, lg[:, ::-1])
    ties = lg[:, 0] == lg[:, 1]
    assert np.array_equal(d2[~ties], 1 - d[~ties])
    assert np.all(d2[ties] == 0)


@pytest.mark.parametrize("arch", ARCHS)
def test_batch_and_thread_independence(arch):
    blob = inputs.weights(arch, 3)
    raw = inputs.device_trace("bing_i", 1500, seed=6)["raw"]
    lg, d = oracle.infer_raw(arch, blob, raw, nthreads=1)
    lga, da = oracle.infer_raw(arch, blob, raw[:700], nthreads=1)
    lgb, db = oracle.infer_raw(arch, blob, raw[700:], nthreads=1)
    assert np.array_equal(lg, np.concatenate([lga, lgb]))
    assert np.array_equal(d, np.concatenate([da, db]))
    lgt, dt = oracle.infer_raw(arch, blob, raw, nthreads=0)
    assert np.array_equal(lg, lgt) and np.array_equal(d, dt)


def test_hidden_unit_permutation():
    # integer weights: permuting hidden units of the first layer (rows of W0/b0 and the
    # matching columns of W_out) is exact; random float weights: within 1e-5.
    rng = np.random.default_rng(9)
    x = oracle.digitize(inputs.edge_raw(3000, seed=8)).astype(np.float32)
    W0 = rng.integers(-3, 4, size=(4, 31)).astype(np.float32)
    b0 = rng.integers(-3, 4, size=4).astype(np.float32)
    W1 = rng.integers(-3, 4, size=(2, 4)).astype(np.float32)
    b1 = rng.integers(-3, 4, size=2).astype(np.float32)
    perm = rng.permutation(4)
    a = np.concatenate([W0.ravel(), b0, W1.ravel(), b1])
    b = np.concatenate([W0[perm].ravel(), b0[perm], W1[:, perm].ravel(), b1])
    assert np.array_equal(oracle.mlp([31, 4, 2], a, x)[0], oracle.mlp([31, 4, 2], b, x)[0])
    blob = inputs.weights(0, 4)
    (W0, b0), (Wo, bo) = _slices(0, blob)
    perm = rng.permutation(256)
    pb = np.concatenate([W0[perm].ravel(), b0[perm], Wo[:, perm].ravel(), bo])
    l1, _ = oracle.mlp([31, 256, 2], blob, x)
    l2, _ = oracle.mlp([31, 256, 2], pb, x)
    rms = np.sqrt((l1.astype(np.float64) ** 2).mean())
    assert np.max(np.abs(l1 - l2)) < 1e-5 * max(rms, 1.0)


def test_infer_digits_equals_infer_raw():
    raw = inputs.edge_raw(1000, seed=12)
    blob = inputs.weights(1, 0)
    a = oracle.infer_raw(1, blob, raw)
    b = oracle.infer_digits(1, blob, oracle.digitize(raw))
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
