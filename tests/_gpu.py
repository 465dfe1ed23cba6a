"""Helpers for the -m gpu parity tests (inputs from the shared generators; expected values from oracle/)."""
import numpy as np
import torch

import oracle
import paper_conf_icpp_chenbpbyo22_b200 as atos
from paper_conf_icpp_chenbpbyo22_b200 import gen

DEV = "cuda:0"


def csr_of(rp, ci, num_parts=1, host=False):
    rpt = torch.from_numpy(np.ascontiguousarray(rp, dtype=np.int64))
    cit = torch.from_numpy(np.ascontiguousarray(ci, dtype=np.int32))
    if not host:
        rpt, cit = rpt.to(DEV), cit.to(DEV)
    return atos.CSR(rpt, cit, device=0, num_parts=num_parts)


def as_u32(t):
    return t.cpu().numpy().view(np.uint32)


def check_pr(rp, ci, rank, st, eps, alpha=0.85, ref=None):
    """Tolerances of BASELINE.json north_star: every rank within 1e-4 relative and
    L1(normalised) <= 1e-5 at eps=1e-6; plus the proven one-sided band and conservation."""
    n = len(rp) - 1
    if ref is None:
        ref, _, ok = oracle.pagerank_jacobi(rp, ci, alpha)
        assert ok
    r = rank.cpu().numpy() if hasattr(rank, "cpu") else rank
    x, xs = r * n, ref * n
    # one-sided: 0 <= x* - x <= eps x*/(1-a)  (+ fp64 rounding slack)
    assert np.all(x <= xs * (1 + 1e-9) + 1e-12), "rank exceeds the fixed point"
    assert np.all(xs - x <= eps * xs / (1 - alpha) * (1 + 1e-6) + 1e-12), "rank below the eps band"
    rel = np.abs(r - ref) / np.maximum(ref, 1e-300)
    assert rel.max() <= 1e-4 or eps > 1e-6
    assert np.abs(r - ref).sum() <= 1e-5 or eps > 1e-6
    deg = np.diff(rp)
    iso = int(np.sum(deg == 0))
    # conservation on symmetric graphs: sum x + sum r/(1-a) = n - a #isolated
    return x.sum() + st["residual_sum"] / (1 - alpha) - (n - alpha * iso)
