"""Pins for the oracle's feature capture (NEXT-1; Fig. 4/5 P:861-932; readings R7-R10).

* hand-worked trace with arrival/completion ties (tests/golden/capture_example.txt);
* the generator's heap-based event simulation (tracesim.c, a different algorithm) on
  synthetic traces of every Table 4 profile;
* invariants: q_now >= 1, q_now <= index-in-device + 1, history latencies match completed
  I/Os, devices are independent (interleaving two devices == capturing each alone).
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden
from paper_conf_asplos_finglertyshar23_b200 import inputs


def _golden():
    rows = read_golden("capture_example.txt")
    dev = np.array([int(r[1].split()[0]) for r in rows], np.int32)
    a = np.array([int(r[1].split()[1]) for r in rows], np.int64)
    c = np.array([int(r[1].split()[2]) for r in rows], np.int64)
    exp = np.array([[int(v) for v in r[2].split()] for r in rows], np.uint32)
    return dev, a, c, exp


def test_hand_worked_capture():
    dev, a, c, exp = _golden()
    assert np.array_equal(oracle.capture(a, c, dev), exp)


@pytest.mark.parametrize("profile", inputs.PROFILE_ORDER)
def test_matches_event_simulation(profile):
    tr = inputs.device_trace(profile, 4000, seed=31, rerate=3.0)
    assert np.array_equal(oracle.capture(tr["arrival_ns"], tr["complete_ns"]), tr["raw"])


def test_devices_are_independent():
    t0 = inputs.device_trace("azure", 1500, seed=1, rerate=3.0)
    t1 = inputs.device_trace("cosmos", 700, seed=2, rerate=3.0)
    a = np.concatenate([t0["arrival_ns"], t1["arrival_ns"]])
    c = np.concatenate([t0["complete_ns"], t1["complete_ns"]])
    d = np.concatenate([np.zeros(1500, np.int32), np.ones(700, np.int32)])
    perm = np.argsort(a, kind="stable")  # interleave by arrival
    out = oracle.capture(a[perm], c[perm], d[perm])
    back = np.empty_like(out)
    back[perm] = out
    assert np.array_equal(back[:1500], t0["raw"])
    assert np.array_equal(back[1500:], t1["raw"])


def test_invariants():
    tr = inputs.device_trace("bing_i", 3000, seed=9, rerate=3.0)
    raw = oracle.capture(tr["arrival_ns"], tr["complete_ns"])
    idx = np.arange(3000)
    assert np.all(raw[:, 0] >= 1) and np.all(raw[:, 0] <= idx + 1)
    lat_all = (tr["complete_ns"] - tr["arrival_ns"]) // 1000
    present = raw[:, 5:9] > 0  # completed I/Os have q_now >= 1, missing history is 0
    assert np.all(np.isin(raw[:, 1:5][present], lat_all))


def test_capture_rows_equals_capture():
    tr = inputs.device_trace("azure", 2500, seed=17, rerate=3.0)
    full = oracle.capture(tr["arrival_ns"], tr["complete_ns"])
    rows = np.array([0, 1, 5, 777, 2499])
    assert np.array_equal(oracle.capture_rows(tr["arrival_ns"], tr["complete_ns"], None, rows),
                          full[rows])
