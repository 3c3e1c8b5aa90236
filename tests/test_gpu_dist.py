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


def _torchrun(script_args, nproc=2):
    env = dict(os.environ, BENCH_SAME_DEVICE="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node",
           str(nproc), "--master-addr", "127.0.0.1", "--master-port", str(_port())] + script_args
    out = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    return [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]


@pytest.mark.parametrize("plan", ["model_affine", "range_split"])
@pytest.mark.parametrize("prec", ["fp32", "f16", "tf32"])
def test_two_rank_cuda_shards_equal_single_process(prec, plan):
    """Per-rank CUDA results of a sharded multi-model batch, gathered to rank 0, equal one
    process's infer_multi over the whole batch bit for bit (decisions and logits); FP32 also
    equals the oracle on a sample. Two ranks share GPU 0 (gloo control plane)."""
    lines = _torchrun(["tests/dist_parity_worker.py", "--prec", prec, "--plan", plan])
    assert len(lines) == 1, lines  # rank 0 alone reports
    r = lines[0]
    assert r["covered_once"] and r["world"] == 2 and min(r["ranks"]) > 0, r
    assert r["decision_mismatches"] == 0 and r["logit_mismatches"] == 0, r
    if prec == "fp32":
        assert r["oracle_mismatches"] == 0 and r["oracle_sample"] > 1000, r


def test_bench_two_ranks_gathers_and_checks_decisions():
    """bench.py --gpus 2 gathers every rank's decisions to rank 0 after the timed region and
    checks them against a single-rank infer_multi of the whole batch."""
    env = dict(os.environ, BENCH_SAME_DEVICE="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2",
           "--steps", "3", "--warmup", "3", "--dist-backend", "gloo", "--no-cpu", "--no-e2e",
           "--n-ios", str(1 << 20)]
    out = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    d = json.loads([l for l in out.stdout.splitlines() if l.startswith("{")][0])
    par = d["multi_rank_parity"]
    assert par["checked"] == 1 << 20 and par["decision_mismatches"] == 0, par
