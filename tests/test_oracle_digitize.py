"""Pins for the oracle's digitisation (readings R1-R6).

Pinned against things other than the oracle itself: hand-worked examples
(tests/golden/digitize_examples.txt), and an exhaustive round trip that rebuilds the
value from the digits (sum d_i * 10^(w-1-i) == min(v, 10^w - 1)) for every v in
[0, 10^5] — the oracle extracts digits by repeated division, the check multiplies back.
"""
import numpy as np
import pytest

import oracle
from conftest import read_golden


def _golden():
    out = []
    for name, rec, dig, s in read_golden("digitize_examples.txt"):
        out.append((name, [int(v) for v in rec.split()], [int(v) for v in dig.split()], int(s)))
    return out


@pytest.mark.parametrize("name,rec,digits,dsum", _golden())
def test_hand_worked_examples(name, rec, digits, dsum):
    got = oracle.digitize(np.array([rec], dtype=np.uint32))[0]
    assert got.tolist() == digits, name
    assert int(got.sum()) == dsum


def _field_digits(digits31):
    """Split the 31 digits back into the 9 fields by the R6 layout."""
    widths = [3, 4, 4, 4, 4, 3, 3, 3, 3]
    fields, pos = [], 0
    for w in widths:
        fields.append(digits31[..., pos:pos + w])
        pos += w
    return fields, widths


def test_exhaustive_round_trip():
    v = np.arange(0, 100_001, dtype=np.uint32)
    raw = np.repeat(v[:, None], 9, axis=1)
    d = oracle.digitize(raw).astype(np.int64)
    assert d.min() >= 0 and d.max() <= 9
    fields, widths = _field_digits(d)
    for f, w in zip(fields, widths):
        back = (f * (10 ** np.arange(w - 1, -1, -1, dtype=np.int64))).sum(axis=1)
        assert np.array_equal(back, np.minimum(v.astype(np.int64), 10 ** w - 1))


def test_fields_are_independent_and_ordered():
    # each field lands only in its own slots (catches a swapped field order)
    for field in range(9):
        rec = np.zeros((1, 9), dtype=np.uint32)
        rec[0, field] = 7
        d = oracle.digitize(rec)[0]
        widths = [3, 4, 4, 4, 4, 3, 3, 3, 3]
        last = sum(widths[:field + 1]) - 1  # least significant digit of that field
        expect = np.zeros(31, dtype=np.uint8)
        expect[last] = 7
        assert d.tolist() == expect.tolist(), field


def test_saturation_extremes():
    rec = np.full((1, 9), 2**32 - 1, dtype=np.uint32)
    assert oracle.digitize(rec)[0].tolist() == [9] * 31
