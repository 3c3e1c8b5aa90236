"""Helpers for the -m gpu parity tests: device placement and comparison metrics.

Inputs come from the seeded generators (paper_conf_asplos_finglertyshar23_b200.inputs);
expected values come ONLY from oracle/ (never from the CUDA path)."""
import numpy as np
import torch

from paper_conf_asplos_finglertyshar23_b200 import lake

DEV = 0


def cuda(a: np.ndarray) -> torch.Tensor:
    if a.dtype == np.uint32:
        a = a.view(np.int32)
    return torch.from_numpy(np.ascontiguousarray(a)).to(f"cuda:{DEV}")


def run_infer(arch_model_id, raw_or_digits: np.ndarray, flags: int, logits=True):
    n = raw_or_digits.shape[0]
    x = cuda(raw_or_digits)
    dec = torch.full((n,), 7, dtype=torch.uint8, device=f"cuda:{DEV}")
    lg = torch.full((n, 2), float("nan"), dtype=torch.float32, device=f"cuda:{DEV}") if logits else None
    lake.infer(x, flags, n, arch_model_id, dec, lg)
    torch.cuda.synchronize()
    return (lg.cpu().numpy() if logits else None), dec.cpu().numpy()


def run_multi(raw: np.ndarray, model_ids: np.ndarray, flags: int, split_calls=False):
    n = raw.shape[0]
    x = cuda(raw)
    ids = cuda(model_ids.astype(np.int32))
    dec = torch.full((n,), 7, dtype=torch.uint8, device=f"cuda:{DEV}")
    lg = torch.full((n, 2), 12345.0, dtype=torch.float32, device=f"cuda:{DEV}")
    wsb = lake.workspace_bytes(n)
    ws = torch.empty(max(wsb, 1), dtype=torch.uint8, device=f"cuda:{DEV}")
    if split_calls:
        lake.multi_group(n, ids, ws, wsb)
        lake.multi_grouped(x, flags, n, dec, lg, ws, wsb)
    else:
        lake.infer_multi(x, flags, n, ids, dec, lg, ws, wsb)
    unk = lake.multi_status(ws, wsb)
    torch.cuda.synchronize()
    return lg.cpu().numpy(), dec.cpu().numpy(), unk


def tc_metrics(lg, dec, ref_lg, ref_dec):
    """S19/S20 metrics: relative error |d| / max(|ref|, rms(ref)), agreement, and the
    largest |logit0 - logit1| (oracle) among disagreements."""
    ref = ref_lg.astype(np.float64)
    rms = np.sqrt(np.mean(ref ** 2))
    rel = np.abs(lg.astype(np.float64) - ref) / np.maximum(np.abs(ref), rms)
    agree = dec == ref_dec
    margin = np.abs(ref[:, 0] - ref[:, 1])
    max_dis_margin = float(margin[~agree].max()) if (~agree).any() else 0.0
    return dict(max_rel=float(rel.max()), agreement=float(agree.mean()),
                max_disagree_margin=max_dis_margin, margin_sd=float(np.std(ref[:, 1] - ref[:, 0])))
