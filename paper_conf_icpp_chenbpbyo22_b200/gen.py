"""Seeded synthetic graph generators (shared by the tests, the bench and the oracle legs).

This module holds NONE of the method's arithmetic: it only builds CSR inputs
shaped like the paper's datasets (Table 2).  It runs unchanged on
CPU or CUDA torch tensors and yields bit-identical graphs on both, because the
only randomness is a counter-based 32-bit hash (``lowbias32``) evaluated with
int64 arithmetic that never overflows (products are split into 16-bit halves),
and the CSR build is sort + unique (unique result).

Recipes:
 * RMAT / Kronecker (Graph500 initiator a,b,c,d = .57,.19,.19,.05): EF * 2^S
   pairs; level l of pair i draws h(seed, l, i); symmetrise, drop self loops,
   dedupe, then a seeded vertex-ID permutation (hubs not clustered at low IDs).
 * mesh: R x C 4-neighbour lattice, row-major IDs (spatially meaningful like
   road_usa); optional bond percolation (keep bond with probability p).
 * torus: R x C 4-regular wraparound lattice (PageRank closed form x = 1).
"""
from __future__ import annotations

import hashlib
from dataclasses import dataclass

import numpy as np
import torch

M32 = 0xFFFFFFFF


def _mul32(x, c: int):
    """(x * c) mod 2^32 for x in [0, 2^32) without int64 overflow."""
    lo, hi = c & 0xFFFF, c >> 16
    return (x * lo + (((x * hi) & 0xFFFF) << 16)) & M32


def lowbias32(x):
    """Chris Wellons' lowbias32 integer hash on values in [0, 2^32) (int or int64 tensor)."""
    x = x ^ (x >> 16)
    x = _mul32(x, 0x7FEB352D)
    x = x ^ (x >> 15)
    x = _mul32(x, 0x846CA68B)
    x = x ^ (x >> 16)
    return x


def hash32(seed: int, stream: int, i):
    """Counter-based 32-bit hash of (seed, stream, counter i < 2^63)."""
    k = lowbias32(((seed & M32) ^ lowbias32((stream * 0x9E3779B9 + (seed >> 32)) & M32)) & M32)
    hi = lowbias32(((i >> 32) ^ k) & M32)
    return lowbias32(((i & M32) ^ hi) & M32)


@dataclass
class Graph:
    """CSR graph: row_ptr int64[n+1], col int32[m] (torch tensors, same device)."""
    n: int
    m: int
    row_ptr: torch.Tensor
    col: torch.Tensor
    name: str = ""

    def to(self, device):
        return Graph(self.n, self.m, self.row_ptr.to(device), self.col.to(device), self.name)

    def numpy(self):
        return self.row_ptr.cpu().numpy(), self.col.cpu().numpy()

    def degrees(self):
        return self.row_ptr[1:] - self.row_ptr[:-1]

    def stats(self) -> dict:
        """Table-2-style row: V, E, max/avg degree, isolated count (+ sha256)."""
        deg = self.degrees()
        return {
            "name": self.name, "V": self.n, "E": self.m,
            "max_degree": int(deg.max().item()) if self.n else 0,
            "avg_degree": (self.m / self.n) if self.n else 0.0,
            "isolated": int((deg == 0).sum().item()),
        }

    def sha256(self) -> str:
        h = hashlib.sha256()
        h.update(self.row_ptr.cpu().numpy().tobytes())
        h.update(self.col.cpu().numpy().tobytes())
        return h.hexdigest()


def _csr_from_sorted_keys(keys: torch.Tensor, n: int, device) -> tuple[torch.Tensor, torch.Tensor]:
    """keys = u*n + v sorted ascending and unique -> (row_ptr, col)."""
    u = keys // n
    col = (keys - u * n).to(torch.int32)
    counts = torch.bincount(u, minlength=n)
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    return row_ptr, col


def csr_from_edges(n: int, src: torch.Tensor, dst: torch.Tensor, symmetric: bool = True,
                   device=None) -> Graph:
    """Symmetrise (optional), drop self loops, dedupe, sort -> CSR."""
    device = device or src.device
    src = src.to(device=device, dtype=torch.int64)
    dst = dst.to(device=device, dtype=torch.int64)
    if symmetric:
        src, dst = torch.cat([src, dst]), torch.cat([dst, src])
    keep = src != dst
    keys = torch.unique(src[keep] * n + dst[keep], sorted=True)
    rp, col = _csr_from_sorted_keys(keys, n, device)
    return Graph(n, int(col.numel()), rp, col)


def permutation(n: int, seed: int, device) -> torch.Tensor:
    """Seeded random permutation: new_id[v]. Sort by (hash>>1, v) -- unique keys -> deterministic."""
    v = torch.arange(n, dtype=torch.int64, device=device)
    key = ((hash32(seed, 0x5EED, v) >> 1) << 32) | v
    order = torch.argsort(key)
    new_id = torch.empty_like(order)
    new_id[order] = v
    return new_id


def rmat(scale: int, edge_factor: int, seed: int, device="cpu", a=0.57, b=0.19, c=0.19,
         permute: bool = True, chunk_pairs: int = 1 << 24, buckets: int | None = None,
         name: str | None = None, rows: tuple[int, int] | None = None) -> Graph:
    """Graph500-initiator RMAT/Kronecker graph, symmetric, no self loops, deduped, ID-permuted.

    Pair i, level l: h = hash32(seed, l, i); quadrant (0,0) if h < a*2^32,
    (0,1) if < (a+b)*2^32, (1,0) if < (a+b+c)*2^32, else (1,1); bit (S-1-l).

    rows = (v_begin, v_end): build only those rows (one rank's 1D block, for the multi-process path) --
    every pair is still drawn, so the rows are bit-identical to the same rows of the full graph; the
    result's row_ptr has v_end - v_begin + 1 entries (starting at 0) and col holds GLOBAL ids; n stays
    the global vertex count.
    """
    device = torch.device(device)
    n = 1 << scale
    npairs = edge_factor * n
    t1 = int(a * 2**32)
    t2 = int((a + b) * 2**32)
    t3 = int((a + b + c) * 2**32)
    new_id = permutation(n, seed ^ 0xA5A5A5A5, device) if permute else None
    if buckets is None:
        buckets = 1 if npairs <= (1 << 26) else 16
    bshift = max(scale - int(np.log2(buckets)), 0)
    parts = [[] for _ in range(buckets)]
    for start in range(0, npairs, chunk_pairs):
        i = torch.arange(start, min(start + chunk_pairs, npairs), dtype=torch.int64, device=device)
        u = torch.zeros_like(i)
        w = torch.zeros_like(i)
        for lvl in range(scale):
            h = hash32(seed, lvl, i)
            bit = 1 << (scale - 1 - lvl)
            ub = h >= t2                       # lower half: quadrants (1,0),(1,1)
            wb = ((h >= t1) & (h < t2)) | (h >= t3)
            u |= ub.to(torch.int64) * bit
            w |= wb.to(torch.int64) * bit
            del h
        if permute:
            u, w = new_id[u], new_id[w]
        keep = u != w
        u, w = u[keep], w[keep]
        su = torch.cat([u, w])
        sw = torch.cat([w, u])
        if rows is not None:
            mine = (su >= rows[0]) & (su < rows[1])
            su, sw = su[mine], sw[mine]
        keys = su * n + sw
        if buckets == 1:
            parts[0].append(keys)
        else:
            bid = su >> bshift
            order = torch.argsort(bid)
            keys, bid = keys[order], bid[order]
            cnt = torch.bincount(bid, minlength=buckets).cpu().tolist()
            off = 0
            for bk in range(buckets):
                if cnt[bk]:
                    parts[bk].append(keys[off:off + cnt[bk]].clone())
                off += cnt[bk]
            del order, bid
        del i, u, w, su, sw, keys
    uniq = []
    for bk in range(buckets):
        if parts[bk]:
            k = torch.cat(parts[bk])
            parts[bk] = None
            uniq.append(torch.unique(k, sorted=True))
            del k
    keys = torch.cat(uniq) if uniq else torch.zeros(0, dtype=torch.int64, device=device)
    del uniq
    nm = name or f"rmat-s{scale}-ef{edge_factor}-seed{seed}"
    if rows is not None:
        vb, ve = rows
        u = keys // n
        col = (keys - u * n).to(torch.int32)
        counts = torch.bincount(u - vb, minlength=ve - vb)
        rp = torch.zeros(ve - vb + 1, dtype=torch.int64, device=device)
        rp[1:] = torch.cumsum(counts, 0)
        return Graph(n, int(col.numel()), rp, col, nm + f"-rows{vb}-{ve}")
    rp, col = _csr_from_sorted_keys(keys, n, device)
    return Graph(n, int(col.numel()), rp, col, nm)


def mesh(R: int, C: int, keep_prob: float = 1.0, seed: int = 0, device="cpu",
         torus: bool = False, name: str | None = None) -> Graph:
    """4-neighbour lattice, row-major ids v = r*C + c; neighbours listed in ascending id order.

    keep_prob < 1: each undirected bond survives iff hash32(seed, 7, bond_id) < p*2^32,
    bond_id = 2*v (bond to the right) or 2*v+1 (bond downward).
    """
    device = torch.device(device)
    n = R * C
    v = torch.arange(n, dtype=torch.int64, device=device)
    r, c = v // C, v % C
    thr = int(keep_prob * 2**32)

    def bond_ok(bid):
        if keep_prob >= 1.0:
            return torch.ones_like(bid, dtype=torch.bool)
        return hash32(seed, 7, bid) < thr

    if torus:
        if R < 3 or C < 3:
            raise ValueError("torus needs R, C >= 3")
        up = ((r - 1) % R) * C + c
        dn = ((r + 1) % R) * C + c
        lf = r * C + (c - 1) % C
        rt = r * C + (c + 1) % C
        ok_up = bond_ok(2 * up + 1)
        ok_dn = bond_ok(2 * v + 1)
        ok_lf = bond_ok(2 * lf)
        ok_rt = bond_ok(2 * v)
    else:
        up, dn, lf, rt = v - C, v + C, v - 1, v + 1
        ok_up = (r > 0) & bond_ok(2 * (v - C).clamp(min=0) + 1)
        ok_dn = (r < R - 1) & bond_ok(2 * v + 1)
        ok_lf = (c > 0) & bond_ok(2 * (v - 1).clamp(min=0))
        ok_rt = (c < C - 1) & bond_ok(2 * v)
    nb = torch.stack([up, lf, rt, dn], dim=1)
    ok = torch.stack([ok_up, ok_lf, ok_rt, ok_dn], dim=1)
    if torus:
        # wraparound breaks ascending order; sort each row of 4
        nb_s, idx = torch.sort(torch.where(ok, nb, torch.full_like(nb, 1 << 62)), dim=1)
        ok = torch.gather(ok, 1, idx)
        nb = nb_s
    counts = ok.sum(dim=1)
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    col = nb[ok].to(torch.int32)
    nm = name or (f"{'torus' if torus else 'mesh'}-{R}x{C}" + (f"-p{keep_prob}-seed{seed}" if keep_prob < 1 else ""))
    return Graph(n, int(col.numel()), row_ptr, col, nm)


def pick_source(g: Graph, seed: int) -> int:
    """Seeded choice among non-isolated vertices (DESIGN.md R-BFS-7)."""
    return pick_source_from_degrees(g.degrees(), seed)


def pick_source_from_degrees(deg: torch.Tensor, seed: int) -> int:
    """pick_source given the (global) degree vector -- e.g. gathered from the ranks' row blocks."""
    cand = torch.nonzero(deg > 0).flatten()
    if cand.numel() == 0:
        return 0
    k = int(hash32(seed, 0x50C, 0)) % int(cand.numel())
    return int(cand[k].item())


def mesh_centre_source(g: Graph, R: int, C: int) -> int:
    """Centre vertex (R//2, C//2), or the nearest non-isolated vertex in ID order after it."""
    deg = g.degrees().cpu()
    v = (R // 2) * C + (C // 2)
    while v < g.n and deg[v] == 0:
        v += 1
    return v if v < g.n else 0


# ---------------------------------------------------------------------------
# The five BASELINE.json configurations
# ---------------------------------------------------------------------------

CONFIGS = {
    "C1": dict(kind="rmat", scale=16, edge_factor=16, seed=1, src_seed=101),
    "C2": dict(kind="mesh", R=4900, C=4900, keep_prob=1.0, seed=2),
    "C2road": dict(kind="mesh", R=4900, C=4900, keep_prob=0.6, seed=2),
    "C3": dict(kind="rmat", scale=22, edge_factor=16, seed=3),
    "C4": dict(kind="rmat", scale=20, edge_factor=64, seed=4),
    "C5": dict(kind="rmat", scale=26, edge_factor=16, seed=5, src_seed=105),
}


def make_config(name: str, device="cpu", **over) -> Graph:
    cfg = dict(CONFIGS[name])
    cfg.update(over)
    kind = cfg.pop("kind")
    cfg.pop("src_seed", None)
    if kind == "rmat":
        return rmat(cfg["scale"], cfg["edge_factor"], cfg["seed"], device=device, name=name)
    return mesh(cfg["R"], cfg["C"], cfg.get("keep_prob", 1.0), cfg.get("seed", 0), device=device, name=name)
