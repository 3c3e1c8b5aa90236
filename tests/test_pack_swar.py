"""The grouping pass's packed digit rows (SWAR form in csrc/digitize.cuh) against the oracle.

pack_record turns a raw record into 31 digit nibbles in the tensor-core slot order
 with multiply-shift digit extraction on two 16-bit lanes at once. The
harness runs that exact function on the host (it is __host__ __device__); this test unpacks
each nibble to its canonical digit position and compares with oracle.digitize, which
extracts digits by repeated division (readings R1-R6): every latency value 0..10050,
every queue value 0..1050 (so the v*41>>12 and v*5243>>19 quotient shortcuts are checked
over their whole clamped domain and past the caps), and random records up to 2^32-1.
"""
import os
import shutil
import subprocess

import numpy as np
import pytest

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _slot_digit(s):  # tc_slot_digit, restated from its definition in DESIGN.md §2
    if s < 16:
        return 3 + s
    if s < 26:
        g = (s - 16) // 2
        return (1 if g == 0 else 17 + 3 * g) + (s & 1)
    if s < 31:
        return 0 if s == 26 else 16 + 3 * (s - 26)
    return 31


@pytest.fixture(scope="module")
def harness(tmp_path_factory):
    nvcc = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(nvcc):
        pytest.skip("nvcc not available")
    exe = str(tmp_path_factory.mktemp("swar") / "pack_swar")
    subprocess.run([nvcc, "-std=c++17", "-O2", "-o", exe, os.path.join(ROOT, "tests", "pack_swar_host.cu")],
                   check=True, capture_output=True)
    return exe


def _pack(exe, raw, tmp_path):
    src, dst = tmp_path / "raw.bin", tmp_path / "packed.bin"
    np.ascontiguousarray(raw, dtype=np.uint32).tofile(src)
    subprocess.run([exe, str(src), str(dst)], check=True)
    return np.fromfile(dst, dtype=np.uint32).reshape(-1, 4)


def _unpack(packed):
    nib = np.zeros((packed.shape[0], 32), dtype=np.uint8)
    for s in range(32):
        nib[:, s] = (packed[:, s // 8] >> np.uint32(4 * (s % 8))) & 0xF
    canon = np.zeros((packed.shape[0], 32), dtype=np.uint8)
    for s in range(32):
        canon[:, _slot_digit(s)] = nib[:, s]
    return canon


def test_pack_record_matches_oracle_digits(harness, tmp_path):
    v = np.arange(0, 10_051, dtype=np.uint32)
    raw = np.zeros((v.size, 9), dtype=np.uint32)
    raw[:, 1:5] = v[:, None]                                   # every latency value
    raw[:, [0, 5, 6, 7, 8]] = (v % 1051)[:, None]              # every queue value
    raw[:, 2] = (v * 7 + 3) % 10_051                           # decorrelate the lanes
    raw[:, 6] = (v * 13 + 5) % 1051
    rng = np.random.default_rng(77)
    big = rng.integers(0, 2**32, size=(4096, 9), dtype=np.uint64).astype(np.uint32)
    big[::3] %= 12_000
    raw = np.concatenate([raw, big, np.full((1, 9), 0xFFFFFFFF, np.uint32)])
    canon = _unpack(_pack(harness, raw, tmp_path))
    want = oracle.digitize(raw)
    np.testing.assert_array_equal(canon[:, :31], want)
    assert np.all(canon[:, 31] == 1)  # slot 31: the constant 1 carrying b0
