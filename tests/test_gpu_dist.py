"""bench.py's multi-rank path on one GPU: torchrun with 2 ranks, gloo control plane, both
ranks on GPU 0 (BENCH_SAME_DEVICE=1). Checks the JSON contract, the shard plan and that the
whole-job value counts every rank's I/Os."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_bench_two_ranks_one_gpu():
    env = dict(os.environ, BENCH_SAME_DEVICE="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2",
           "--steps", "3", "--warmup", "3", "--dist-backend", "gloo", "--no-cpu", "--no-e2e",
           "--n-ios", str(1 << 20)]
    out = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["steps"] == 3
    assert d["config"]["n_ios"] == 1 << 20
    assert d["value"] > 0 and d["gpu_launches"] > 0
    assert d["config"]["plan"] in ("model_affine", "range_split")
