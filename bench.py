#!/usr/bin/env python
"""bench.py — batched LinnOS I/O-latency classification on B200 (LAKE's hot path).

Metric (BASELINE.json): I/O inferences/s (and batch latency vs batch size, `--mode sweep`),
1/2/4/8 B200, % of roofline. Default workload = BASELINE.json configs[4] ("C5"): 64 per-SSD
NN+2 models, 2^24 interleaved I/Os, sharded across the ranks (strong scaling: the total is
fixed). A step = one pass of the whole hot path over the rank's shard: model grouping
(histogram / scan / scatter) + fused digitise -> 4 layers -> argmax on tcgen05 tensor cores
(fp16 operands, fp32 accumulation), through the C ABI (lake_linnos_infer_multi).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--prec f16]
    torchrun --nproc-per-node N bench.py --gpus N ...
    python bench.py --impl reference ...     # the CPU oracle on the same workload
    python bench.py --mode sweep             # C2 latency vs batch size (writes JSON lines)

Inputs are synthetic and seeded (paper_conf_asplos_finglertyshar23_b200.inputs); weights
are random init (no trained LinnOS weights are published). The oracle is executed only in
the cpu_baseline leg and under --impl reference.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_asplos_finglertyshar23_b200 import inputs, shard  # noqa: E402

ARCH_NAME = {0: "NN (31-256-2)", 1: "NN+1 (31-256-256-2)", 2: "NN+2 (31-256-256-256-2)"}
# algorithmic FLOP per I/O, 2 per MAC, no padding
ARCH_FLOPS = {0: 2 * (31 * 256 + 256 * 2), 1: 2 * (31 * 256 + 256 * 256 + 256 * 2),
              2: 2 * (31 * 256 + 2 * 256 * 256 + 256 * 2)}
RAW_BYTES = 36
NN_OTC_CYCLES_PER_TILE = 2 * 128.1 + 16 * 62.1  # NN fp16/bf16 tile on the tensor pipe (DESIGN 6.3)
L2_BYTES = 126 * 1024 * 1024
THROTTLE_BAD = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown")


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="C5", choices=["C1", "C3", "C4", "C5"])
    p.add_argument("--prec", default=None, choices=["fp32", "f16", "bf16", "tf32"])
    p.add_argument("--arch", type=int, default=None)
    p.add_argument("--n-ios", dest="n", type=int, default=None)
    p.add_argument("--mode", default="throughput", choices=["throughput", "sweep", "report", "family"])
    p.add_argument("--sweep-out", default=None)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--no-latency", action="store_true",
                   help="skip the compact latency-vs-batch block of the default line")
    p.add_argument("--cpu-seconds", type=float, default=12.0)
    p.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                   help="control-plane backend (gloo: lets a 1-GPU box run several ranks)")
    return p.parse_args()


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ------------------------------------------------------------------ distributed plumbing
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def dist_init(world, local, backend="nccl"):
    import torch
    import torch.distributed as dist
    if world > 1 and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if backend == "nccl":
            torch.cuda.set_device(local)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    return dist if world > 1 else None


def max_over_ranks(x: float, dist, device=None) -> float:
    if dist is None:
        return x
    import torch
    if dist.get_backend() == "gloo":
        device = None  # gloo reduces host tensors
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier(dist):
    if dist is not None:
        dist.barrier()


# ------------------------------------------------------------------ clocks (pynvml)
class ClockSampler:
    """Samples SM clock and throttle reasons every 10 ms during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
        0x100: "display_clock_setting",
    }

    def __init__(self, index: int):
        self.ok = False
        self.samples, self.reasons = [], 0
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.reasons |= int(self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
            except Exception:
                pass
            time.sleep(0.01)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        names = [v for k, v in self.REASONS.items() if self.reasons & k and v != "gpu_idle"]
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": int(self.max_mhz),
                "reasons": names, "samples": len(self.samples)}


# ------------------------------------------------------------------ workload
def workload(args, world, rank):
    cfg = inputs.CONFIGS[args.config]
    n = args.n or cfg["n"]
    arch = cfg["arch"] if args.arch is None else args.arch
    t = time.time()
    w = inputs.workload(args.config, n=n, arch=arch)
    log(f"[rank {rank}] generated {args.config} n={n} arch={arch} in {time.time() - t:.1f}s")
    raw, ids = w["raw"], w["model_ids"]
    n_models = cfg["models"]
    p = shard.plan(ids, n_models, world)
    if p["kind"] == "model_affine":
        idx = shard.rank_indices(ids, p["owner"], rank)
        mine = [m for m in range(n_models) if p["owner"][m] == rank]
    else:
        b, e = shard.range_split(n, world, rank)
        idx = np.arange(b, e)
        mine = list(range(n_models))
    return dict(raw=np.ascontiguousarray(raw[idx]), ids=np.ascontiguousarray(ids[idx]), idx=idx,
                plan_obj=p, models={m: w["models"][m] for m in mine}, n_total=n, arch=arch,
                n_models=n_models, plan=p["kind"], imbalance=p["imbalance"],
                full_raw=raw, full_ids=ids, all_models=w["models"])


def config_obj(args, wl, prec, world, copies):
    n = wl["n_total"]
    return {
        "workload": (f"{args.config}: {wl['n_models']} per-SSD {ARCH_NAME[wl['arch']].split()[0]} "
                     f"model(s), {n} interleaved synthetic I/Os"
                     + (", sharded across ranks (strong scaling)" if world > 1 else "")),
        "n_ios": n, "models": wl["n_models"], "arch": ARCH_NAME[wl["arch"]],
        "path": {"fp32": "CUDA-core FP32 (bit-exact)", "f16": "tcgen05 cta_group::2, fp16 in / fp32 acc",
                 "bf16": "tcgen05 cta_group::2, bf16 in / fp32 acc",
                 "tf32": "tcgen05 cta_group::2 kind::tf32, tf32 in / fp32 acc"}[prec],
        "input": "raw records (36 B/IO), digitised in-kernel; decisions out (1 B/IO)",
        "api": "lake_linnos_infer_multi (group + fused MLP)",
        "plan": wl["plan"], "imbalance": round(wl["imbalance"], 4),
        "l2": (f"inputs larger than L2 ({copies} rotating input copies per rank, "
               f">= 2x126 MB)" if copies > 1 else "inputs larger than L2"),
    }


# ------------------------------------------------------------------ CPU oracle timing
def time_oracle(wl, seconds: float):
    """The oracle, as it stands, on a bounded deterministic stride sample of the workload,
    all host cores. Returns dict(value I/O-per-s, cores, sample)."""
    import oracle
    raw, ids, models = wl["full_raw"], wl["full_ids"], wl["all_models"]
    cores = oracle.max_threads()
    probe = np.arange(0, raw.shape[0], max(1, raw.shape[0] // 512))[:512]
    t0 = time.perf_counter()
    oracle.infer_multi_raw(models, raw[probe], ids[probe], nthreads=0)
    per = (time.perf_counter() - t0) / probe.size
    s = int(min(raw.shape[0], max(1024, seconds / max(per, 1e-9))))
    stride = max(1, raw.shape[0] // s)
    idx = np.arange(0, raw.shape[0], stride)[:s]
    t0 = time.perf_counter()
    oracle.infer_multi_raw(models, raw[idx], ids[idx], nthreads=0)
    dt = time.perf_counter() - t0
    return dict(value=idx.size / dt, unit="inferences/s", cores=cores, kind="oracle",
                sample=(f"stride-{stride} sample of {idx.size} of the {raw.shape[0]} I/Os "
                        f"({len(models)} models), {dt:.1f} s wall on {cores} threads"))


# ------------------------------------------------------------------ latency vs batch (compact)
LAT_SIZES = (1, 2, 4, 8, 16, 64, 1024, 4096)


def latency_vs_batch(lake, local: int, reps: int = 200, warm: int = 20):
    """BASELINE's second metric in the default line: batch latency vs batch size (Fig. 8,
    PAPER.md P:1288-1311) for NN and NN+2 on a compact grid. Per (arch, path, b): end to end
    through the public host-buffer call lake_linnos_infer_host (pinned host records in,
    decisions out, stream sync; host clock, median and p99 of `reps`) and device-only (CUDA
    events around `reps` launches of lake_linnos_infer on resident inputs); the 1-thread
    oracle for the same batch; the crossover b (reading R22: smallest b whose GPU end-to-end
    median beats the 1-thread oracle); and the persistent FP32 server at b = 1."""
    import torch
    import oracle
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    raw_all = inputs.device_trace("azure", max(LAT_SIZES), 1200, 1.0)["raw"]
    out = {"sizes": list(LAT_SIZES), "unit": "us", "archs": {}}
    with ClockSampler(local) as clk:
        for arch in (0, 2):
            blob = inputs.weights(arch, 0)
            mid = 40 + arch
            lake.load_weights(mid, arch, blob, local)
            rec = {}
            cpu = []
            for b in LAT_SIZES:
                raw = np.ascontiguousarray(raw_all[:b])
                oreps = max(1, min(50, int(2e4 / (b * (1 + 15 * arch)))))
                best = float("inf")
                for _ in range(5 if b <= 64 else 1):  # best of 5 blocks: host-noise robust
                    t0 = time.perf_counter()
                    for _ in range(oreps):
                        oracle.infer_raw(arch, blob, raw, nthreads=1)
                    best = min(best, (time.perf_counter() - t0) * 1e6 / oreps)
                cpu.append(round(best, 2))
            rec["cpu_1thread_us"] = cpu
            for prec in ("fp32", "f16"):
                flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
                e2e, p99, devus = [], [], []
                for b in LAT_SIZES:
                    raw = np.ascontiguousarray(raw_all[:b])
                    h_in = torch.from_numpy(raw.view(np.int32)).pin_memory()
                    h_dec = torch.empty(b, dtype=torch.uint8).pin_memory()
                    d_in = h_in.to(dev)
                    d_dec = torch.empty(b, dtype=torch.uint8, device=dev)
                    stb = lake.host_staging_bytes(b, flags)
                    stg = torch.empty(stb, dtype=torch.uint8, device=dev)
                    for _ in range(warm):
                        lake.infer_host(h_in, flags, b, mid, None, h_dec, None, stg, stb, stream)
                    ts = []
                    for _ in range(reps):
                        t0 = time.perf_counter()
                        lake.infer_host(h_in, flags, b, mid, None, h_dec, None, stg, stb, stream)
                        ts.append((time.perf_counter() - t0) * 1e6)
                    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    ev0.record(stream)
                    for _ in range(reps):
                        lake.infer(d_in, flags, b, mid, d_dec, None, stream)
                    ev1.record(stream)
                    torch.cuda.synchronize()
                    e2e.append(round(float(np.median(ts)), 2))
                    p99.append(round(float(np.percentile(ts, 99)), 2))
                    devus.append(round(ev0.elapsed_time(ev1) * 1e3 / reps, 2))
                cross = next((b for b, g, c in zip(LAT_SIZES, e2e, cpu) if g < c), None)
                rec[prec] = {"e2e_us_median": e2e, "e2e_us_p99": p99, "device_us": devus,
                             "crossover_batch": cross}
            sdec = np.zeros(1, np.uint8)
            raw1 = np.ascontiguousarray(raw_all[:1])
            with lake.Server(mid) as srv:
                for _ in range(warm):
                    srv.infer(raw1, 1, sdec)
                st = []
                for _ in range(reps):
                    t0 = time.perf_counter()
                    srv.infer(raw1, 1, sdec)
                    st.append((time.perf_counter() - t0) * 1e6)
            rec["server_fp32_b1_us_median"] = round(float(np.median(st)), 2)
            rec["server_crossover"] = 1 if float(np.median(st)) < cpu[0] else None
            out["archs"][ARCH_NAME[arch]] = rec
            lake.unload(mid, local)
    out["clocks"] = clk.summary()
    out["paper_context"] = ("A100 through LAKE, Fig. 8: GPU profitable for batches > 8 (NN), "
                            "> 3 (NN+1), > 2 (NN+2); PAPER.md P:1296-1311, Table 3 P:1088")
    out["how"] = ("e2e: lake_linnos_infer_host (pinned host buffers; zero-copy for b <= 2^14) "
                  "median of %d after %d warm-up; device: CUDA events over %d lake_linnos_infer "
                  "launches; cpu: oracle on 1 host thread" % (reps, warm, reps))
    return out


# ------------------------------------------------------------------ our implementation
def run_ours(args):
    import torch
    world, rank, local = dist_env()
    if args.gpus != world and world > 1:
        log(f"warning: --gpus {args.gpus} but WORLD_SIZE {world}")
    # testing aid: BENCH_SAME_DEVICE=1 puts every rank on GPU 0 (with --dist-backend gloo)
    if os.environ.get("BENCH_SAME_DEVICE") == "1":
        local = 0
    dist = dist_init(world, local, args.dist_backend)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    from paper_conf_asplos_finglertyshar23_b200 import lake

    wl = workload(args, world, rank)
    prec = args.prec or "f16"
    flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
    for m, (arch, blob) in wl["models"].items():
        lake.load_weights(m, arch, blob, local)
    n = wl["raw"].shape[0]
    shard_bytes = n * RAW_BYTES
    copies = max(1, math.ceil(2 * L2_BYTES / max(shard_bytes, 1))) if shard_bytes < 2 * L2_BYTES else 1
    raw_np = wl["raw"].view(np.int32)
    xs = [torch.from_numpy(raw_np).to(dev) for _ in range(copies)]
    ids = torch.from_numpy(wl["ids"]).to(dev)
    dec = torch.empty(max(n, 1), dtype=torch.uint8, device=dev)
    wsb = lake.workspace_bytes(n)
    ws = torch.empty(max(wsb, 1), dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def step(i):
        lake.infer_multi(xs[i % copies], flags, n, ids, dec, None, ws, wsb, stream)

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    barrier(dist)
    torch.cuda.synchronize()
    lake.reset_launch_count()
    lake.profile_enable(True)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for i in range(args.steps):
            step(i)
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier(dist)
    torch.cuda.synchronize()
    launches = lake.launch_count()
    kern_ms, kern_n = lake.profile_read()
    lake.profile_enable(False)
    ms = ev0.elapsed_time(ev1)
    ms_max = max_over_ranks(ms, dist, dev)
    kern_avg = kern_ms / max(kern_n, 1)
    kern_avg_max = max_over_ranks(kern_avg, dist, dev)
    n_max = max_over_ranks(float(n), dist, dev)
    value = wl["n_total"] * args.steps / (ms_max / 1e3)

    # ---- multi-rank parity (outside the timed region): every rank's decisions, gathered to
    # rank 0, must equal one rank's infer_multi over the whole batch (independent I/Os, one
    # model per block device: PAPER.md Fig. 4 caption P:906-909) -----------------------------
    parity = None
    if dist is not None:
        step(0)
        torch.cuda.synchronize()
        gathered = [None] * world
        dist.all_gather_object(gathered, (wl["idx"], dec[:n].cpu().numpy()))
        if rank == 0:
            for m, (arch, blob) in wl["all_models"].items():
                if m not in wl["models"]:
                    lake.load_weights(m, arch, blob, local)
            N = wl["n_total"]
            fx = torch.from_numpy(wl["full_raw"].view(np.int32)).to(dev)
            fids = torch.from_numpy(wl["full_ids"]).to(dev)
            fdec = torch.empty(N, dtype=torch.uint8, device=dev)
            fwsb = lake.workspace_bytes(N)
            fws = torch.empty(fwsb, dtype=torch.uint8, device=dev)
            lake.infer_multi(fx, flags, N, fids, fdec, None, fws, fwsb, stream)
            torch.cuda.synchronize()
            ref = fdec.cpu().numpy()
            seen = np.zeros(N, dtype=np.int64)
            bad = 0
            for ridx, rdec in gathered:
                seen[ridx] += 1
                bad += int((rdec != ref[ridx]).sum())
            parity = {"checked": int((seen == 1).sum()), "decision_mismatches": bad,
                      "covered_once": bool(np.all(seen == 1)),
                      "reference": "single-rank lake_linnos_infer_multi of the whole batch on rank 0",
                      "how": "per-rank decisions all-gathered after the timed region"}
            del fx, fids, fdec, fws
        barrier(dist)

    # ---- roofline of the dominant kernel (fused MLP) -------------------------------------
    peaks = {}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            peaks = json.load(f)
    except Exception:
        pass
    if prec == "fp32":
        # FP32 CUDA-core peak derived from the guide's unit counts
        sm_mhz = peaks.get("sm_max_mhz", 1965.0)
        peak, src = 148 * 128 * 2 * sm_mhz * 1e6 / 1e12, "derived: 148 SM x 128 FFMA x 2 x max clock"
        bound = "alu"
    else:
        peak = peaks.get("bf16_tflops")
        src = "measured (MEASURED_PEAKS.json bf16 burst; fp16:bf16 nominal ratio 1:1)"
        if peak is None:
            peak, src = 1590.0, "fallback (B200_PROFILING.md)"
        if prec == "tf32":
            peak, src = peak / 2, src.replace("fp16:bf16 nominal ratio 1:1", "x tf32:bf16 nominal ratio 1:2")
        bound = "tensor"
    flops_launch = ARCH_FLOPS[wl["arch"]] * n_max
    achieved = flops_launch / (kern_avg_max / 1e3) / 1e12
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        try:
            with open(tpath) as f:
                tj = json.load(f)
            key = f"{args.config}_{prec}_g{world}"
            traffic = tj.get(key)
        except Exception:
            traffic = None
    roofline = {"bound": bound, "achieved": round(achieved, 2), "peak": round(peak, 1),
                "unit": "TFLOP/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                "kernel": "mlp_tc_kernel" if prec != "fp32" else "mlp_fp32_kernel",
                "kernel_ms": round(kern_avg_max, 4), "flops_per_launch": flops_launch,
                "peak_source": src,
                "kernel_share_of_step": round(kern_avg_max / (ms_max / args.steps), 4)}

    # ---- end to end through the C ABI with host buffers ----------------------------------
    e2e = None
    if not args.no_e2e:
        h_in = torch.from_numpy(raw_np).pin_memory()
        # one-byte model ids when every id fits (LAKE_IDS_U8): the path is PCIe-bound
        ids_np = wl["ids"]
        narrow = ids_np.size > 0 and int(ids_np.min()) >= 0 and int(ids_np.max()) < 256
        id_bytes = 1 if narrow else 4
        eflags = flags | (lake.LAKE_IDS_U8 if narrow else 0)
        h_ids = torch.from_numpy(ids_np.astype(np.uint8) if narrow else ids_np).pin_memory()
        h_dec = torch.empty(max(n, 1), dtype=torch.uint8).pin_memory()
        stb = lake.host_staging_bytes(n, eflags)
        stg = torch.empty(max(stb, 1), dtype=torch.uint8, device=dev)
        e_steps = max(1, min(args.steps, 5))
        lake.infer_host(h_in, eflags, n, -1, h_ids, h_dec, None, stg, stb, stream)
        barrier(dist)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(e_steps):
            lake.infer_host(h_in, eflags, n, -1, h_ids, h_dec, None, stg, stb, stream)
        e_ms = (time.perf_counter() - t0) * 1e3 / e_steps
        e_ms = max_over_ranks(e_ms, dist, dev)
        e2e = {"value": round(wl["n_total"] / (e_ms / 1e3), 1), "unit": "inferences/s",
               "h2d_bytes_per_step": int(n * (RAW_BYTES + id_bytes)), "d2h_bytes_per_step": int(n),
               "ms_per_step": round(e_ms, 3),
               "how": f"lake_linnos_infer_host: pinned H2D of raw + {id_bytes}-byte ids, group+fused MLP, D2H "
                      "of decisions, stream sync; host wall clock, max over ranks"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = time_oracle(wl, args.cpu_seconds)
        cpu["value"] = round(cpu["value"], 1)
    latency = None
    if rank == 0 and world == 1 and not args.no_latency:
        latency = latency_vs_batch(lake, local)

    if rank == 0:
        line = {
            "metric": "I/O inferences/sec", "value": round(value, 1), "unit": "inferences/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms_max / args.steps, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": prec,
            "data": "synthetic (seeded traces shaped like PAPER.md Table 4; random-init weights)",
            "config": config_obj(args, wl, prec, world, copies),
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "multi_rank_parity": parity,
            "latency": latency,
            "gpu_launches": int(launches), "clocks": clk.summary(),
            # context, not the target (BASELINE.json north_star): the paper's claim and the
            # hardware it was measured on; beside it, this run's reduction vs the oracle
            "paper_context": {
                "claim": "ML-backed I/O latency predictor inference time reduced by up to 96% "
                         "(95% in the introduction) with GPU acceleration through LAKE",
                "hardware": "2x 16-core Intel Xeon Gold 6226R, NVIDIA A100, Linux 6.0 kernel space",
                "citation": "PAPER.md P:74-75 (abstract), P:183-184 (Section 1), P:1064-1068 (testbed)",
                "this_run_time_reduction_vs_oracle": (
                    round(1.0 - cpu["value"] / value, 6) if cpu and value > 0 else None),
            },
        }
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.destroy_process_group()


# ------------------------------------------------------------------ reference arm (oracle)
def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    import oracle
    cfg = inputs.CONFIGS[args.config]
    n = args.n or cfg["n"]
    arch = cfg["arch"] if args.arch is None else args.arch
    w = inputs.workload(args.config, n=n, arch=arch)
    raw, ids, models = w["raw"], w["model_ids"], w["models"]
    cores = oracle.max_threads()
    # per-step sample sized for ~3 s of oracle work so the whole run takes a few minutes
    probe = np.arange(0, n, max(1, n // 256))[:256]
    t0 = time.perf_counter()
    oracle.infer_multi_raw(models, raw[probe], ids[probe], nthreads=0)
    per = (time.perf_counter() - t0) / probe.size
    s = int(min(n, max(256, 3.0 / max(per, 1e-9))))
    stride = max(1, n // s)
    idx = np.arange(0, n, stride)[:s]
    r, i_ = raw[idx], ids[idx]
    for _ in range(args.warmup):
        oracle.infer_multi_raw(models, r, i_, nthreads=0)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.infer_multi_raw(models, r, i_, nthreads=0)
    dt = time.perf_counter() - t0
    value = idx.size * args.steps / dt
    sample = (f"each step: stride-{stride} sample of {idx.size} of the {n} I/Os of "
              f"{args.config} ({len(models)} models), oracle on {cores} host threads")
    line = {
        "impl": "reference", "metric": "I/O inferences/sec", "value": round(value, 1),
        "unit": "inferences/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(dt * 1e3 / args.steps, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "fp32",
        "data": "synthetic (seeded traces shaped like PAPER.md Table 4; random-init weights)",
        "config": {"workload": f"{args.config}: {len(models)} per-SSD "
                               f"{ARCH_NAME[arch].split()[0]} model(s), {n} I/Os (sampled per step)",
                   "n_ios": n, "models": len(models), "arch": ARCH_NAME[arch]},
        "cpu_baseline": {"value": round(value, 1), "unit": "inferences/s", "cores": cores,
                         "kind": "oracle", "sample": sample},
        "e2e": {"value": round(value, 1), "unit": "inferences/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ C2: latency sweep
def run_sweep(args):
    """Batch latency vs batch size (BASELINE configs[1], Fig. 8): end-to-end
    (pinned H2D -> infer -> D2H -> sync, host clock) and device-only, per arch x path, and
    the 1-thread oracle for the same batch; crossover = smallest b where GPU e2e < CPU."""
    import torch
    import oracle
    from paper_conf_asplos_finglertyshar23_b200 import lake
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    sizes = [1 << k for k in range(13)]
    raw_all = inputs.device_trace("azure", max(sizes), 1200, 1.0)["raw"]
    out = []
    for arch in (0, 1, 2):
        blob = inputs.weights(arch, 0)
        lake.load_weights(40 + arch, arch, blob, 0)
        for prec in ("fp32", "f16", "bf16", "tf32"):
            flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
            cross = None
            gcross = None
            scross = None
            for b in sizes:
                raw = np.ascontiguousarray(raw_all[:b])
                h_in = torch.from_numpy(raw.view(np.int32)).pin_memory()
                h_dec = torch.empty(b, dtype=torch.uint8).pin_memory()
                d_in = torch.from_numpy(raw.view(np.int32)).to(dev)
                d_dec = torch.empty(b, dtype=torch.uint8, device=dev)
                stb = lake.host_staging_bytes(b, flags)
                stg = torch.empty(stb, dtype=torch.uint8, device=dev)
                reps, warm = 200, 20

                def once():  # the public host-buffer call: H2D, fused kernel, D2H, sync
                    lake.infer_host(h_in, flags, b, 40 + arch, None, h_dec, None, stg, stb, stream)
                for _ in range(warm):
                    once()
                ts = []
                for _ in range(reps):
                    t0 = time.perf_counter()
                    once()
                    ts.append((time.perf_counter() - t0) * 1e6)
                # CUDA-Graph variant (C2): H2D copy, fused kernel and D2H copy captured once,
                # each batch one graph replay + stream sync (launch overheads amortised)
                gs = torch.cuda.Stream()
                g_dec = torch.empty(b, dtype=torch.uint8).pin_memory()
                with torch.cuda.stream(gs):
                    lake.infer(d_in, flags, b, 40 + arch, d_dec, None, gs)  # warm (attributes)
                gs.synchronize()
                graph = torch.cuda.CUDAGraph()
                with torch.cuda.graph(graph, stream=gs):
                    d_in.copy_(h_in, non_blocking=True)
                    lake.infer(d_in, flags, b, 40 + arch, d_dec, None, gs)
                    g_dec.copy_(d_dec, non_blocking=True)
                gt = []
                with torch.cuda.stream(gs):  # replay() launches on the current stream
                    for _ in range(warm):
                        graph.replay()
                        gs.synchronize()
                    for _ in range(reps):
                        t0 = time.perf_counter()
                        graph.replay()
                        gs.synchronize()
                        gt.append((time.perf_counter() - t0) * 1e6)
                if not np.array_equal(g_dec.numpy(), h_dec.numpy()):
                    raise RuntimeError(f"graph replay differs from infer_host (arch {arch} {prec} b={b})")
                del graph
                ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ev0.record(stream)
                for _ in range(reps):
                    lake.infer(d_in, flags, b, 40 + arch, d_dec, None, stream)
                ev1.record(stream)
                torch.cuda.synchronize()
                dev_us = ev0.elapsed_time(ev1) * 1e3 / reps
                # 1-thread oracle for the same batch
                oreps = max(1, min(50, int(2e4 / (b * (1 + 15 * arch)))))
                t0 = time.perf_counter()
                for _ in range(oreps):
                    oracle.infer_raw(arch, blob, raw, nthreads=1)
                cpu_us = (time.perf_counter() - t0) * 1e6 / oreps
                med = float(np.median(ts))
                gmed = float(np.median(gt))
                if cross is None and med < cpu_us:
                    cross = b
                if gcross is None and gmed < cpu_us:
                    gcross = b
                row = dict(arch=ARCH_NAME[arch], prec=prec, batch=b, e2e_us_median=round(med, 2),
                           e2e_us_p99=round(float(np.percentile(ts, 99)), 2),
                           graph_us_median=round(gmed, 2),
                           graph_us_p99=round(float(np.percentile(gt, 99)), 2),
                           device_us=round(dev_us, 2), cpu_1thread_us=round(cpu_us, 2))
                if prec == "fp32" and b <= lake.LAKE_SERVER_MAX_BATCH:
                    # NEXT-2: persistent resident-weights server (doorbell, no launch/copies)
                    sdec = np.zeros(b, np.uint8)
                    with lake.Server(40 + arch) as srv:
                        for _ in range(warm):
                            srv.infer(raw, b, sdec)
                        st = []
                        for _ in range(reps):
                            t0 = time.perf_counter()
                            srv.infer(raw, b, sdec)
                            st.append((time.perf_counter() - t0) * 1e6)
                    row["server_us_median"] = round(float(np.median(st)), 2)
                    row["server_us_p99"] = round(float(np.percentile(st, 99)), 2)
                    if scross is None and row["server_us_median"] < cpu_us:
                        scross = b
                out.append(row)
                log(json.dumps(row))
            out.append(dict(arch=ARCH_NAME[arch], prec=prec, crossover_batch=cross,
                            graph_crossover_batch=gcross,
                            **({"server_crossover_batch": scross} if prec == "fp32" else {})))
            log(json.dumps(out[-1]))
        lake.unload(40 + arch, 0)
    path = args.sweep_out or os.path.join(ROOT, "gpurun_out", "sweep.jsonl")
    os.makedirs(os.path.dirname(path), exist_ok=True)
    with open(path, "w") as f:
        for r in out:
            f.write(json.dumps(r) + "\n")
    print(json.dumps({"metric": "batch latency vs batch size (C2)", "rows": len(out),
                      "crossovers": [r for r in out if "crossover_batch" in r]}))


# ------------------------------------------------------------------ C3 / C4 report
def run_report(args):
    """BASELINE configs[2] (C3: NN+1 / NN+2, 2^20 I/Os, tensor cores vs FP32), configs[3]
    (C4: 3 per-SSD models interleaved, 2^22 I/Os, every arch, grouping overhead) and
    configs[4] on one GPU (C5: 64 NN+2 models, 2^24 I/Os, fp16 / bf16 / FP32): throughput,
    fraction of the relevant peak, and accuracy against the oracle on a sample."""
    import torch
    import oracle
    from paper_conf_asplos_finglertyshar23_b200 import lake
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    tpeak = peaks.get("bf16_tflops", 1590.0)
    fpeak = 148 * 128 * 2 * peaks.get("sm_max_mhz", 1965.0) * 1e6 / 1e12
    rows = []

    def peak_of(prec):
        return fpeak if prec == "fp32" else (tpeak / 2 if prec == "tf32" else tpeak)

    def peak_label(prec):
        if prec == "fp32":
            return "FP32 %.1f TF/s (derived from unit counts)" % fpeak
        if prec == "tf32":
            return "tf32 %.1f TF/s = measured bf16 %.1f x nominal tf32:bf16 1:2" % (tpeak / 2, tpeak)
        return "bf16 %.1f TF/s (measured; fp16 same nominal rate)" % tpeak

    def timed(fn, reps=10):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(reps):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps

    # ---- C3
    n = 1 << 20
    raw = inputs.workload("C3", n=n)["raw"]
    x = torch.from_numpy(raw.view(np.int32)).to(dev)
    dec = torch.empty(n, dtype=torch.uint8, device=dev)
    lg = torch.empty((n, 2), dtype=torch.float32, device=dev)
    smp = np.random.default_rng(0).choice(n, 8192, replace=False)
    for arch in (1, 2):
        blob = inputs.weights(arch, 0)
        lake.load_weights(60 + arch, arch, blob, 0)
        rlg, rdec = oracle.infer_raw(arch, blob, raw[smp], nthreads=0)
        ref = rlg.astype(np.float64)
        rms = np.sqrt(np.mean(ref ** 2))
        for prec in ("fp32", "f16", "bf16", "tf32"):
            flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
            ms = timed(lambda: lake.infer(x, flags, n, 60 + arch, dec, lg, stream))
            lake.infer(x, flags, n, 60 + arch, dec, lg, stream)
            torch.cuda.synchronize()
            d = dec.cpu().numpy()[smp]
            l = lg.cpu().numpy()[smp].astype(np.float64)
            rel = np.abs(l - ref) / np.maximum(np.abs(ref), rms)
            dis = d != rdec
            tflops = ARCH_FLOPS[arch] * n / (ms / 1e3) / 1e12
            rows.append(dict(config="C3", arch=ARCH_NAME[arch], path=prec, n=n,
                             ms=round(ms, 4), inferences_per_s=round(n / (ms / 1e3), 1),
                             tflops=round(tflops, 2),
                             frac_of_peak=round(tflops / peak_of(prec), 4), peak=peak_label(prec),
                             sample=int(smp.size), agreement=float(1 - dis.mean()),
                             max_rel_err=float(rel.max()),
                             max_disagree_margin=float(np.abs(ref[dis, 0] - ref[dis, 1]).max()) if dis.any() else 0.0,
                             margin_sd=float(np.std(ref[:, 1] - ref[:, 0]))))
            log(json.dumps(rows[-1]))
        lake.unload(60 + arch, 0)
    # ---- C4: 3 per-SSD models interleaved, every arch (headline NN+2 fp16)
    n = 1 << 22
    for arch in (2, 1, 0):
        w = inputs.workload("C4", n=n, arch=arch)
        x = torch.from_numpy(w["raw"].view(np.int32)).to(dev)
        ids = torch.from_numpy(w["model_ids"]).to(dev)
        dec = torch.empty(n, dtype=torch.uint8, device=dev)
        wsb = lake.workspace_bytes(n)
        ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
        for m, (a, blob) in w["models"].items():
            lake.load_weights(m, a, blob, 0)
        flags = lake.LAKE_IN_RAW | lake.LAKE_PREC_F16
        t_multi = timed(lambda: lake.infer_multi(x, flags, n, ids, dec, None, ws, wsb, stream))
        t_group = timed(lambda: lake.multi_group(n, ids, ws, wsb, stream))
        mids = w["model_ids"]
        parts = [torch.from_numpy(np.ascontiguousarray(w["raw"][mids == m]).view(np.int32)).to(dev)
                 for m in range(3)]
        t_split = timed(lambda: [lake.infer(p, flags, p.shape[0], m, dec, None, stream)
                                 for m, p in enumerate(parts)])
        rows.append(dict(config="C4", arch=ARCH_NAME[arch], path="f16", n=n, models=3,
                         infer_multi_ms=round(t_multi, 4), group_ms=round(t_group, 4),
                         presplit_3_infer_ms=round(t_split, 4),
                         inferences_per_s=round(n / (t_multi / 1e3), 1),
                         grouping_overhead=round(t_multi / t_split - 1, 4)))
        log(json.dumps(rows[-1]))
        if arch == 0:
            # single-model NN over 2^24 I/Os (the C4 records four times over: > 2x L2),
            # the model LinnOS deploys, per tensor-core type
            big = torch.from_numpy(np.ascontiguousarray(np.tile(w["raw"], (4, 1))).view(np.int32)).to(dev)
            dbig = torch.empty(1 << 24, dtype=torch.uint8, device=dev)
            for prec in ("f16", "bf16", "tf32"):
                fl = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
                ms = timed(lambda: lake.infer(big, fl, 1 << 24, 0, dbig, None, stream))
                tflops = ARCH_FLOPS[0] * (1 << 24) / (ms / 1e3) / 1e12
                gbs = (RAW_BYTES + 1) * (1 << 24) / (ms / 1e3) / 1e9
                row = dict(config="C4-single", arch="NN", path=prec, n=1 << 24, ms=round(ms, 4),
                           inferences_per_s=round((1 << 24) / (ms / 1e3), 1),
                           tflops=round(tflops, 2), frac_of_peak=round(tflops / peak_of(prec), 4),
                           peak=peak_label(prec), hbm_gb_s=round(gbs, 1))
                if prec in ("f16", "bf16"):
                    # NN's tensor-core bound is the MMA instruction rate, not FLOPs: per 256-row
                    # tile 2 layer-0 MMAs (N=256, 128.1 cycles) + 16 output-layer MMAs (N=16,
                    # 62.1 cycles: the per-instruction floor, scripts/microbench/umma_dep.cu),
                    # tiles spread over 74 CTA pairs, at the SM max clock
                    tiles_per_pair = ((1 << 24) // 256 + 73) // 74
                    bound_ms = NN_OTC_CYCLES_PER_TILE * tiles_per_pair / (peaks.get("sm_max_mhz", 1965.0) * 1e3)
                    row.update(mma_instr_bound_ms=round(bound_ms, 4),
                               frac_of_mma_instr_bound=round(bound_ms / ms, 4))
                rows.append(row)
                log(json.dumps(rows[-1]))
            del big, dbig
        for m in w["models"]:
            lake.unload(m, 0)
        del x, ids, dec, ws, parts
    # ---- C5 on one GPU: 64 NN+2 models interleaved, 2^24 I/Os, every path (the throughput
    # mode times the fp16 headline; here fp16, bf16 and FP32 with oracle-sample accuracy)
    n = 1 << 24
    w = inputs.workload("C5", n=n)
    x = torch.from_numpy(w["raw"].view(np.int32)).to(dev)
    ids = torch.from_numpy(w["model_ids"]).to(dev)
    dec = torch.empty(n, dtype=torch.uint8, device=dev)
    lg = torch.empty((n, 2), dtype=torch.float32, device=dev)
    wsb = lake.workspace_bytes(n)
    ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
    for m, (a, blob) in w["models"].items():
        lake.load_weights(m, a, blob, 0)
    smp = np.random.default_rng(5).choice(n, 8192, replace=False)
    mids = w["model_ids"][smp]
    rlg = np.zeros((smp.size, 2), np.float32)
    rdec = np.zeros(smp.size, np.uint8)
    for m in np.unique(mids):
        sel = mids == m
        rlg[sel], rdec[sel] = oracle.infer_raw(2, w["models"][int(m)][1], w["raw"][smp[sel]], nthreads=0)
    ref = rlg.astype(np.float64)
    rms = np.sqrt(np.mean(ref ** 2))
    for prec in ("f16", "bf16", "tf32", "fp32"):
        flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[prec]
        ms = timed(lambda: lake.infer_multi(x, flags, n, ids, dec, lg, ws, wsb, stream),
                   reps=10 if prec != "fp32" else 3)
        lake.infer_multi(x, flags, n, ids, dec, lg, ws, wsb, stream)
        torch.cuda.synchronize()
        d = dec.cpu().numpy()[smp]
        l = lg.cpu().numpy()[smp].astype(np.float64)
        rel = np.abs(l - ref) / np.maximum(np.abs(ref), rms)
        dis = d != rdec
        tflops = ARCH_FLOPS[2] * n / (ms / 1e3) / 1e12
        rows.append(dict(config="C5", arch=ARCH_NAME[2], path=prec, n=n, models=64,
                         ms=round(ms, 4), inferences_per_s=round(n / (ms / 1e3), 1),
                         tflops=round(tflops, 2),
                         frac_of_peak=round(tflops / peak_of(prec), 4), peak=peak_label(prec),
                         api="infer_multi (group + fused MLP), logits written",
                         sample=int(smp.size), agreement=float(1 - dis.mean()),
                         bit_exact_logits=bool(np.array_equal(l.astype(np.float32).view(np.uint32),
                                                              rlg.view(np.uint32))),
                         max_rel_err=float(rel.max()),
                         max_disagree_margin=float(np.abs(ref[dis, 0] - ref[dis, 1]).max()) if dis.any() else 0.0))
        log(json.dumps(rows[-1]))
    path = args.sweep_out or os.path.join(ROOT, "gpurun_out", "report.jsonl")
    os.makedirs(os.path.dirname(path), exist_ok=True)
    with open(path, "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    print(json.dumps({"metric": "C3/C4/C5 report", "rows": len(rows)}))


# ------------------------------------------------------------------ NEXT-4 MLP family
FP32_PEAK_TFLOPS = 74.4  # 148 SM x 128 FP32 lanes x 2 FLOP x 1.965 GHz


def run_family(args):
    """NEXT-4: the MLLB / KML-shaped MLPs (include/lake_mlp.h, readings
    R25-R28). Per model: batch latency vs batch size 1..1024 (Fig. 10 / Fig. 11's range,
    P:1436-1535): end to end through the public call with pinned host buffers
    (lake_mlp_infer_host: the kernel reads the features from and writes the classes to host
    memory, then a stream sync) and device-only (CUDA events), beside the 1-thread oracle for the same batch, with the crossover batch; then
    throughput at 2^24 rows (inputs resident in HBM, larger than L2) against the FP32 and
    HBM rooflines, and the oracle on all host cores on a bounded sample."""
    import torch
    import oracle
    from paper_conf_asplos_finglertyshar23_b200 import lake
    from paper_conf_asplos_finglertyshar23_b200.inputs import family
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    pk = os.path.join(ROOT, "MEASURED_PEAKS.json")
    peaks = json.load(open(pk)) if os.path.exists(pk) else {}
    hbm_peak = float(peaks.get("hbm_gbs", 7700.0))
    hbm_src = "measured (MEASURED_PEAKS.json hbm_gbs)" if "hbm_gbs" in peaks else "nominal fallback"
    rows = []
    for mid, (name, cfg) in enumerate(sorted(family.FAMILY.items())):
        widths, act = cfg["widths"], cfg["act"]
        blob = family.weights(widths, 0)
        lake.mlp_load(mid, widths, act, blob, 0)
        C = widths[-1]
        x_all = family.features(1 << 24, widths[0], 3000 + mid)
        cross = None
        for b in [1 << k for k in range(11)]:
            x = np.ascontiguousarray(x_all[:b])
            h_x = torch.from_numpy(x).pin_memory()
            h_c = torch.empty(b, dtype=torch.int32).pin_memory()
            d_x = h_x.to(dev)
            d_c = torch.empty(b, dtype=torch.int32, device=dev)
            reps, warm = 200, 20

            def once():  # the public host-buffer call (zero-copy for pinned buffers)
                lake.mlp_infer_host(h_x, b, mid, h_c, None, None, 0, stream)
            for _ in range(warm):
                once()
            ts = []
            for _ in range(reps):
                t0 = time.perf_counter()
                once()
                ts.append((time.perf_counter() - t0) * 1e6)
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            for _ in range(reps):
                lake.mlp_infer(d_x, b, mid, d_c, None, stream)
            ev1.record(stream)
            torch.cuda.synchronize()
            dev_us = ev0.elapsed_time(ev1) * 1e3 / reps
            _, rc = oracle.mlp_family(widths, act, blob, x, nthreads=1)
            if not np.array_equal(h_c.numpy(), rc) and act == family.ACT_RELU:
                raise RuntimeError(f"{name} b={b}: classes differ from the oracle")
            oreps = max(1, min(200, int(2e5 / b)))
            t0 = time.perf_counter()
            for _ in range(oreps):
                oracle.mlp_family(widths, act, blob, x, nthreads=1)
            cpu_us = (time.perf_counter() - t0) * 1e6 / oreps
            med = float(np.median(ts))
            if cross is None and med < cpu_us:
                cross = b
            row = dict(model=name, widths=list(widths), act=["relu", "sigmoid"][act], batch=b,
                       e2e_us_median=round(med, 2), e2e_us_p99=round(float(np.percentile(ts, 99)), 2),
                       device_us=round(dev_us, 2), cpu_1thread_us=round(cpu_us, 2))
            rows.append(row)
            log(json.dumps(row))
        # throughput at 2^24 rows
        n = 1 << 24
        d_x = torch.from_numpy(x_all).to(dev)
        d_c = torch.empty(n, dtype=torch.int32, device=dev)
        for _ in range(max(3, args.warmup)):
            lake.mlp_infer(d_x, n, mid, d_c, None, stream)
        K = max(5, args.steps)
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        for _ in range(K):
            lake.mlp_infer(d_x, n, mid, d_c, None, stream)
        ev1.record(stream)
        torch.cuda.synchronize()
        ms = ev0.elapsed_time(ev1) / K
        fma = sum(widths[l] * widths[l + 1] for l in range(len(widths) - 1))
        byt = 4 * widths[0] + 4
        tflops = n * 2 * fma / (ms * 1e-3) / 1e12
        gbps = n * byt / (ms * 1e-3) / 1e9
        samp = np.arange(0, n, 64)
        t0 = time.perf_counter()
        oracle.mlp_family(widths, act, blob, x_all[samp], nthreads=0)
        cpu_s = time.perf_counter() - t0
        row = dict(model=name, widths=list(widths), act=["relu", "sigmoid"][act], n_rows=n,
                   kernel_ms=round(ms, 4), rows_per_s=round(n / (ms * 1e-3), 1),
                   flop_per_row=2 * fma, bytes_per_row=byt,
                   roofline_alu={"achieved": round(tflops, 2), "peak": FP32_PEAK_TFLOPS,
                                 "unit": "TFLOP/s", "frac": round(tflops / FP32_PEAK_TFLOPS, 4),
                                 "peak_source": "derived from unit counts (DESIGN.md §7.1)"},
                   roofline_hbm={"achieved": round(gbps, 1), "peak": hbm_peak, "unit": "GB/s",
                                 "frac": round(gbps / hbm_peak, 4), "peak_source": hbm_src},
                   cpu_baseline={"value": round(len(samp) / cpu_s, 1), "unit": "rows/s",
                                 "cores": oracle.max_threads(), "kind": "oracle",
                                 "sample": f"stride-64 sample of {len(samp)} rows"})
        rows.append(row)
        log(json.dumps(row))
        rows.append(dict(model=name, crossover_batch=cross))
        lake.mlp_unload(mid, 0)
        del d_x, d_c
    path = args.sweep_out or os.path.join(ROOT, "gpurun_out", "family.jsonl")
    os.makedirs(os.path.dirname(path), exist_ok=True)
    with open(path, "w") as f:
        for r in rows:
            f.write(json.dumps(r) + "\n")
    print(json.dumps({"metric": "NEXT-4 MLP family: latency vs batch, throughput", "rows": len(rows),
                      "crossovers": [r for r in rows if "crossover_batch" in r]}))


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    elif args.mode == "sweep":
        run_sweep(args)
    elif args.mode == "report":
        run_report(args)
    elif args.mode == "family":
        run_family(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
