"""Serial CPU oracle for the Atos hot path (ctypes wrapper over liboracle.so).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_icpp_chenbpbyo22_b200`` never
imports it and shares no code with it (the C sources live in this directory
only).  Paper citations (P:<line> of /root/reference/PAPER.md) are in
``atos_oracle.c`` next to each function.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "atos_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

UNREACHED = 0xFFFFFFFF


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc -O2 (single-threaded, no vectorisation flags)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            P = ctypes.c_void_p
            i64, i32, u64, dbl = ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double
            lib.oracle_bfs.argtypes = [i64, P, P, i64, P]
            lib.oracle_bfs.restype = i32
            lib.oracle_validate_bfs.argtypes = [i64, P, P, i64, P]
            lib.oracle_validate_bfs.restype = i32
            lib.oracle_pagerank_jacobi.argtypes = [i64, P, P, dbl, dbl, i32, P, P]
            lib.oracle_pagerank_jacobi.restype = i32
            lib.oracle_pagerank_push.argtypes = [i64, P, P, dbl, dbl, P, P, P]
            lib.oracle_pagerank_push.restype = i32
            lib.oracle_pagerank_residual.argtypes = [i64, P, P, dbl, P, P]
            lib.oracle_pagerank_residual.restype = i32
            lib.oracle_color_greedy.argtypes = [i64, P, P, P, P]
            lib.oracle_color_greedy.restype = i64
            lib.oracle_color_jp.argtypes = [i64, P, P, u64, P]
            lib.oracle_color_jp.restype = i64
            lib.oracle_color_jp_rounds.argtypes = [i64, P, P, u64, P]
            lib.oracle_color_jp_rounds.restype = i64
            lib.oracle_validate_color.argtypes = [i64, P, P, P]
            lib.oracle_validate_color.restype = i32
            lib.oracle_splitmix64.argtypes = [u64]
            lib.oracle_splitmix64.restype = u64
            _lib = lib
    return _lib


def _csr(row_ptr, col):
    rp = np.ascontiguousarray(np.asarray(row_ptr), dtype=np.int64)
    ci = np.ascontiguousarray(np.asarray(col), dtype=np.int32)
    n = rp.shape[0] - 1
    return n, rp, ci


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def bfs(row_ptr, col, src: int) -> np.ndarray:
    """Exact BFS depths (uint32, 0xFFFFFFFF unreachable). See oracle_bfs."""
    n, rp, ci = _csr(row_ptr, col)
    depth = np.empty(n, dtype=np.uint32)
    rc = _load().oracle_bfs(n, _p(rp), _p(ci), int(src), _p(depth))
    if rc != 0:
        raise ValueError("oracle_bfs: bad arguments")
    return depth


def validate_bfs(row_ptr, col, src: int, depth) -> int:
    """Graph500-style validator; 0 = valid."""
    n, rp, ci = _csr(row_ptr, col)
    d = np.ascontiguousarray(depth, dtype=np.uint32)
    return int(_load().oracle_validate_bfs(n, _p(rp), _p(ci), int(src), _p(d)))


def pagerank_jacobi(row_ptr, col, alpha: float = 0.85, tol: float = 1e-13, max_iter: int = 1000):
    """Fixed point x/n of x = (1-a)1 + a P^T x by Jacobi iteration. Returns (rank, iters, converged)."""
    n, rp, ci = _csr(row_ptr, col)
    out = np.empty(n, dtype=np.float64)
    it = ctypes.c_int(0)
    rc = _load().oracle_pagerank_jacobi(n, _p(rp), _p(ci), float(alpha), float(tol), int(max_iter),
                                        _p(out), ctypes.byref(it))
    if rc < 0:
        raise ValueError("oracle_pagerank_jacobi: bad arguments")
    return out, int(it.value), rc == 0


def pagerank_push(row_ptr, col, alpha: float = 0.85, eps: float = 1e-6):
    """Serial Alg.3-init + Alg.4 push PageRank. Returns (rank/n, residue, pops)."""
    n, rp, ci = _csr(row_ptr, col)
    out = np.empty(n, dtype=np.float64)
    res = np.empty(n, dtype=np.float64)
    pops = ctypes.c_int64(0)
    rc = _load().oracle_pagerank_push(n, _p(rp), _p(ci), float(alpha), float(eps), _p(out), _p(res),
                                      ctypes.byref(pops))
    if rc != 0:
        raise ValueError("oracle_pagerank_push: bad arguments")
    return out, res, int(pops.value)


def pagerank_residual(row_ptr, col, x, alpha: float = 0.85) -> np.ndarray:
    """r = (1-a)1 + a P^T x - x for an UNNORMALISED candidate x (x = rank * n). See oracle_pagerank_residual."""
    n, rp, ci = _csr(row_ptr, col)
    xx = np.ascontiguousarray(x, dtype=np.float64)
    if xx.shape[0] != n:
        raise ValueError("pagerank_residual: x must have n entries")
    r = np.empty(n, dtype=np.float64)
    if _load().oracle_pagerank_residual(n, _p(rp), _p(ci), float(alpha), _p(xx), _p(r)) != 0:
        raise ValueError("oracle_pagerank_residual: bad arguments")
    return r


def color_greedy(row_ptr, col, order=None):
    """First-fit greedy in `order` (default vertex-ID order). Returns (color, ncolors)."""
    n, rp, ci = _csr(row_ptr, col)
    color = np.empty(n, dtype=np.int32)
    o = None if order is None else np.ascontiguousarray(order, dtype=np.int64)
    k = _load().oracle_color_greedy(n, _p(rp), _p(ci), None if o is None else _p(o), _p(color))
    if k < 0:
        raise ValueError("oracle_color_greedy failed")
    return color, int(k)


def color_jp(row_ptr, col, seed: int):
    n, rp, ci = _csr(row_ptr, col)
    color = np.empty(n, dtype=np.int32)
    k = _load().oracle_color_jp(n, _p(rp), _p(ci), int(seed) & (2**64 - 1), _p(color))
    if k < 0:
        raise ValueError("oracle_color_jp failed")
    return color, int(k)


def color_jp_rounds(row_ptr, col, seed: int):
    n, rp, ci = _csr(row_ptr, col)
    color = np.empty(n, dtype=np.int32)
    k = _load().oracle_color_jp_rounds(n, _p(rp), _p(ci), int(seed) & (2**64 - 1), _p(color))
    if k < 0:
        raise ValueError("oracle_color_jp_rounds failed")
    return color, int(k)


def validate_color(row_ptr, col, color) -> int:
    """0 = proper colouring with color[v] <= deg(v)."""
    n, rp, ci = _csr(row_ptr, col)
    c = np.ascontiguousarray(color, dtype=np.int32)
    return int(_load().oracle_validate_color(n, _p(rp), _p(ci), _p(c)))


def splitmix64(x: int) -> int:
    return int(_load().oracle_splitmix64(int(x) & (2**64 - 1)))
