"""Multi-rank parity on the CUDA path (launched by tests/test_gpu_dist.py under torchrun).

Each rank scores only its shard of an interleaved multi-model batch through
lake_linnos_infer_multi (model-affine plan: only its own models loaded; range split: every
model loaded), then the per-rank (index, decision, logits) triples are all-gathered to rank
0, which checks that they reassemble, bit for bit, the single-process infer_multi result over
the whole batch — the property that makes sharding without a data-path collective legal
(independent I/Os, one model per block device: PAPER.md Fig. 4 caption).
FP32 results are additionally compared with the oracle on a sample.

usage: torchrun --nproc-per-node 2 tests/dist_parity_worker.py --prec f16 --plan model_affine
(BENCH_SAME_DEVICE=1 puts every rank on GPU 0; the control plane is gloo then.)
"""
import argparse
import json
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_finglertyshar23_b200 import inputs, lake, shard  # noqa: E402

N_MODELS = 6
N = 120_000


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--prec", default="f16", choices=["fp32", "f16", "bf16", "tf32"])
    ap.add_argument("--plan", default="model_affine", choices=["model_affine", "range_split"])
    args = ap.parse_args()
    world, rank = int(os.environ["WORLD_SIZE"]), int(os.environ["RANK"])
    local = 0 if os.environ.get("BENCH_SAME_DEVICE") == "1" else int(os.environ["LOCAL_RANK"])
    dist.init_process_group("gloo")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    raw, mids = inputs.multi_device_trace(N, N_MODELS, seed_base=2600, rerate=3.0)
    ids = (mids + 40).astype(np.int32)  # calibrated slots 40..45, mixed architectures
    models = {40 + m: (m % 3, inputs.weights(m % 3, 40 + m)) for m in range(N_MODELS)}
    p = shard.plan(mids, N_MODELS, world, max_imbalance=1.5)
    if args.plan == "model_affine":
        assert p["kind"] == "model_affine", p
        idx = shard.rank_indices(mids, p["owner"], rank)
        mine = [40 + m for m in range(N_MODELS) if p["owner"][m] == rank]
    else:
        b, e = shard.range_split(N, world, rank)
        idx = np.arange(b, e)
        mine = list(models)
    for m in mine:
        lake.load_weights(m, models[m][0], models[m][1], local)
    flags = lake.LAKE_IN_RAW | lake.PREC_FLAGS[args.prec]

    def run(sel):
        n = sel.size
        x = torch.from_numpy(np.ascontiguousarray(raw[sel]).view(np.int32)).to(dev)
        i = torch.from_numpy(np.ascontiguousarray(ids[sel])).to(dev)
        dec = torch.empty(max(n, 1), dtype=torch.uint8, device=dev)
        lg = torch.empty((max(n, 1), 2), dtype=torch.float32, device=dev)
        wsb = lake.workspace_bytes(n)
        ws = torch.empty(max(wsb, 1), dtype=torch.uint8, device=dev)
        lake.infer_multi(x, flags, n, i, dec, lg, ws, wsb)
        torch.cuda.synchronize(dev)
        return dec.cpu().numpy()[:n], lg.cpu().numpy()[:n]

    dec, lg = run(idx)
    payload = [None] * world
    dist.all_gather_object(payload, (idx, dec, lg))
    result = None
    if rank == 0:
        for m in models:  # the single-process reference: every model on one device
            if m not in mine:
                lake.load_weights(m, models[m][0], models[m][1], local)
        fdec, flg = run(np.arange(N))
        seen = np.zeros(N, dtype=np.int64)
        bad_dec = bad_lg = 0
        for ridx, rdec, rlg in payload:
            seen[ridx] += 1
            bad_dec += int((rdec != fdec[ridx]).sum())
            bad_lg += int((rlg.view(np.uint32) != flg[ridx].view(np.uint32)).any(axis=1).sum())
        result = dict(prec=args.prec, plan=p["kind"] if args.plan == "model_affine" else "range_split",
                      world=world, n=N, covered_once=bool(np.all(seen == 1)),
                      decision_mismatches=bad_dec, logit_mismatches=bad_lg,
                      ranks=[int(r[0].size) for r in payload])
        if args.prec == "fp32":
            import oracle
            smp = np.arange(0, N, 29)
            rlg, rdec = oracle.infer_multi_raw(models, raw[smp], ids[smp], nthreads=0)
            result["oracle_sample"] = int(smp.size)
            result["oracle_mismatches"] = int((rdec != fdec[smp]).sum()) + int(
                (rlg.view(np.uint32) != flg[smp].view(np.uint32)).any(axis=1).sum())
        print(json.dumps(result), flush=True)
    dist.barrier()
    for m in list(models):
        try:
            lake.unload(m, local)
        except lake.LakeError:
            pass
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
