"""B200-native Atos hot path: asynchronous BFS / PageRank / graph colouring on a
single shared lock-free task queue (Chen et al., ICPP'22).

Thin Python binding over the C ABI of ``libatos.so`` (include/atos.h): every
step of the path runs in the library's CUDA kernels; this module only
marshals arguments (torch tensors are used for device memory and streams).
There is no CPU fallback -- if the library cannot be loaded every call raises.
"""
from __future__ import annotations

import ctypes

import torch

from . import _lib
from ._lib import UNREACHED, Stats, default_cfg

__all__ = ["CSR", "bfs", "pagerank", "color", "bfs_bsp", "pagerank_bsp", "color_bsp", "UNREACHED", "launches", "partition_range", "Comm"]


def _ptr(t: torch.Tensor) -> ctypes.c_void_p:
    return ctypes.c_void_p(t.data_ptr())


class CSR:
    """Graph handle (atos_csr).  row_ptr: int64[n+1], col: int32[m], host or CUDA tensors."""

    def __init__(self, row_ptr: torch.Tensor, col: torch.Tensor, device: int = 0, num_parts: int = 1,
                 layout: str = "auto"):
        """layout (atos_csr_create_ex): "auto" -- the degree layout when it pays (large, skewed graphs),
        "degree" -- always, "input" -- keep the caller's ids.  The layout is invisible to callers: ids in
        and out are the caller's."""
        lib = _lib.load()
        row_ptr = row_ptr.contiguous()
        col = col.contiguous()
        if row_ptr.dtype != torch.int64 or col.dtype != torch.int32:
            raise TypeError("row_ptr must be int64 and col int32")
        self.n = int(row_ptr.numel()) - 1
        self.m = int(col.numel())
        self.device = device
        where = _lib.MEM_DEVICE if row_ptr.is_cuda else _lib.MEM_HOST
        if col.is_cuda != row_ptr.is_cuda:
            raise ValueError("row_ptr and col must live in the same memory space")
        h = ctypes.c_void_p()
        flags = {"auto": _lib.LAYOUT_AUTO, "input": _lib.LAYOUT_INPUT, "degree": _lib.LAYOUT_DEGREE}.get(layout)
        if flags is None:
            raise ValueError("layout must be 'auto', 'degree' or 'input'")
        rc = lib.atos_csr_create_ex(ctypes.byref(h), self.n, self.m, _ptr(row_ptr), _ptr(col), where, device,
                                    num_parts, flags)
        _lib.check(rc, "atos_csr_create_ex")
        self._h = h
        self.num_parts = num_parts

    @classmethod
    def from_graph(cls, g, device: int = 0, num_parts: int = 1, layout: str = "auto") -> "CSR":
        return cls(g.row_ptr, g.col, device=device, num_parts=num_parts, layout=layout)

    @classmethod
    def _wrap(cls, handle, n, m, device, num_parts):
        self = cls.__new__(cls)
        self._h, self.n, self.m, self.device, self.num_parts = handle, n, m, device, num_parts
        return self

    @property
    def layout(self) -> str:
        """The layout the library chose at creation: "degree" or "input" (atos_csr_layout)."""
        v = ctypes.c_int()
        _lib.check(_lib.load().atos_csr_layout(self.handle, ctypes.byref(v)), "atos_csr_layout")
        return "degree" if v.value == _lib.LAYOUT_DEGREE else "input"

    @property
    def handle(self):
        if self._h is None:
            raise RuntimeError("CSR handle already closed")
        return self._h

    def close(self):
        if getattr(self, "_h", None) is not None:
            _lib.load().atos_csr_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _run(fn_name: str, g: CSR, out: torch.Tensor, args: tuple, stream, knobs: dict):
    lib = _lib.load()
    st = Stats()
    timeline = knobs.pop("timeline", None)
    cfg = default_cfg(**knobs)
    if timeline is not None:
        if not (timeline.is_cuda and timeline.dtype == torch.int64 and timeline.is_contiguous()):
            raise TypeError("timeline must be a contiguous int64 CUDA tensor of 4*cap entries")
        cfg.timeline = ctypes.c_void_p(timeline.data_ptr())
        cfg.timeline_cap = timeline.numel() // 4
    cfg.stats = ctypes.pointer(st)
    if out.is_cuda:
        cfg.out_where = _lib.MEM_DEVICE
        if stream is None:
            stream = torch.cuda.current_stream(out.device)
    else:
        cfg.out_where = _lib.MEM_HOST
    cfg.stream = ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)
    rc = getattr(lib, fn_name)(g.handle, *args, _ptr(out), ctypes.byref(cfg))
    _lib.check(rc, fn_name)
    return out, st.as_dict()


def _local_len(g: CSR) -> int:
    return getattr(g, "n_local", g.n)


def bfs(g: CSR, src: int, out: torch.Tensor | None = None, stream=None, **knobs):
    """Speculative BFS (Alg.2).  Returns (depth int32 tensor -- reinterpret as uint32, stats)."""
    if out is None:
        out = torch.empty(_local_len(g), dtype=torch.int32, device=f"cuda:{g.device}")
    return _run("atos_bfs", g, out, (int(src),), stream, knobs)


def pagerank(g: CSR, alpha: float = 0.85, eps: float = 1e-6, out: torch.Tensor | None = None, stream=None,
             **knobs):
    """Asynchronous push PageRank (Alg.3 init + Alg.4).  Returns (rank float64 tensor = x/n, stats)."""
    if out is None:
        out = torch.empty(_local_len(g), dtype=torch.float64, device=f"cuda:{g.device}")
    return _run("atos_pagerank", g, out, (float(alpha), float(eps)), stream, knobs)


def color(g: CSR, seed: int = 1, out: torch.Tensor | None = None, stream=None, **knobs):
    """Asynchronous speculative colouring (Alg.6).  Returns (colour int32 tensor, stats)."""
    if out is None:
        out = torch.empty(g.n, dtype=torch.int32, device=f"cuda:{g.device}")
    return _run("atos_color", g, out, (ctypes.c_uint64(seed & (2**64 - 1)),), stream, knobs)


def bfs_bsp(g: CSR, src: int, out: torch.Tensor | None = None, stream=None, **knobs):
    """Bulk-synchronous BFS baseline (Alg.1).  Same result as bfs()."""
    if out is None:
        out = torch.empty(g.n, dtype=torch.int32, device=f"cuda:{g.device}")
    return _run("atos_bfs_bsp", g, out, (int(src),), stream, knobs)


def pagerank_bsp(g: CSR, alpha: float = 0.85, eps: float = 1e-6, out: torch.Tensor | None = None, stream=None,
                 **knobs):
    """Bulk-synchronous PageRank baseline (Alg.3).  Same output scale and bound as pagerank()."""
    if out is None:
        out = torch.empty(g.n, dtype=torch.float64, device=f"cuda:{g.device}")
    return _run("atos_pagerank_bsp", g, out, (float(alpha), float(eps)), stream, knobs)


def color_bsp(g: CSR, seed: int = 1, out: torch.Tensor | None = None, stream=None, **knobs):
    """Bulk-synchronous speculative colouring baseline (Alg.5)."""
    if out is None:
        out = torch.empty(g.n, dtype=torch.int32, device=f"cuda:{g.device}")
    return _run("atos_color_bsp", g, out, (ctypes.c_uint64(seed & (2**64 - 1)),), stream, knobs)


def timeline_table(timeline: torch.Tensor, stats: dict):
    """Samples (t_us from the first sample, done, tail, head) of a cfg.timeline buffer."""
    k = min(int(stats.get("timeline_len", 0)), timeline.numel() // 4)
    t = timeline[: 4 * k].view(k, 4).cpu()
    if k:
        t = t.clone()
        t[:, 0] -= t[0, 0].item()
    return t


def launches() -> int:
    """Number of libatos kernel launches since load."""
    return int(_lib.load().atos_kernel_launches())


def partition_range(n: int, nparts: int, part: int):
    lib = _lib.load(build_if_missing=False) if _lib._lib is None else _lib._lib
    b, e = ctypes.c_int64(), ctypes.c_int64()
    _lib.check(lib.atos_partition_range(n, nparts, part, ctypes.byref(b), ctypes.byref(e)),
               "atos_partition_range")
    return b.value, e.value


class Comm:
    """NCCL communicator of one rank (atos_comm); unique id exchanged by the caller (e.g. torch.distributed)."""

    def __init__(self, nranks: int, rank: int, unique_id: bytes, device: int):
        lib = _lib.load()
        h = ctypes.c_void_p()
        buf = ctypes.create_string_buffer(unique_id, _lib.COMM_ID_BYTES)
        _lib.check(lib.atos_comm_create(ctypes.byref(h), nranks, rank, buf, _lib.COMM_ID_BYTES, device),
                   "atos_comm_create")
        self._h, self.nranks, self.rank, self.device = h, nranks, rank, device

    @classmethod
    def host(cls, nranks: int, rank: int, device: int, group=None) -> "Comm":
        """Host-staged transport (atos_comm_create_host): the exchange rounds' counts/payload all-to-alls and
        termination allreduces run over torch.distributed on CPU tensors of `group` (e.g. gloo).  The library
        still does every step of the path on the GPU; only the bytes between ranks travel through the host."""
        import torch.distributed as dist
        lib = _lib.load()

        def a2a(_user, send, send_bytes, recv, recv_bytes):
            try:
                sb = [int(send_bytes[i]) for i in range(nranks)]
                rb = [int(recv_bytes[i]) for i in range(nranks)]
                src = torch.empty(sum(sb), dtype=torch.uint8)
                if sum(sb):
                    ctypes.memmove(src.data_ptr(), send, sum(sb))
                dst = torch.empty(sum(rb), dtype=torch.uint8)
                dist.all_to_all_single(dst, src, output_split_sizes=rb, input_split_sizes=sb, group=group)
                if sum(rb):
                    ctypes.memmove(recv, dst.data_ptr(), sum(rb))
                return 0
            except Exception:  # noqa: BLE001 -- an exception must not cross the C ABI
                return 1

        def ar(_user, value, dtype):
            try:
                ct = ctypes.c_uint64 if dtype == 0 else ctypes.c_double
                p = ctypes.cast(value, ctypes.POINTER(ct))
                t = torch.tensor([p[0]], dtype=torch.int64 if dtype == 0 else torch.float64)
                dist.all_reduce(t, group=group)
                p[0] = int(t.item()) if dtype == 0 else float(t.item())
                return 0
            except Exception:  # noqa: BLE001
                return 1

        self = cls.__new__(cls)
        self._cbs = (_lib.HOST_A2A_FN(a2a), _lib.HOST_AR_FN(ar))  # kept alive with the communicator
        h = ctypes.c_void_p()
        _lib.check(lib.atos_comm_create_host(ctypes.byref(h), nranks, rank, device, self._cbs[0], self._cbs[1],
                                             None), "atos_comm_create_host")
        self._h, self.nranks, self.rank, self.device = h, nranks, rank, device
        return self

    @staticmethod
    def unique_id() -> bytes:
        lib = _lib.load()
        buf = ctypes.create_string_buffer(_lib.COMM_ID_BYTES)
        _lib.check(lib.atos_comm_unique_id(buf, _lib.COMM_ID_BYTES), "atos_comm_unique_id")
        return buf.raw

    def partition(self, n_global: int, v_begin: int, v_end: int, row_ptr_local: torch.Tensor,
                  col_global: torch.Tensor) -> CSR:
        lib = _lib.load()
        h = ctypes.c_void_p()
        where = _lib.MEM_DEVICE if row_ptr_local.is_cuda else _lib.MEM_HOST
        rp, ci = row_ptr_local.contiguous(), col_global.contiguous()
        _lib.check(lib.atos_csr_create_part(ctypes.byref(h), self._h, n_global, v_begin, v_end, int(ci.numel()),
                                            _ptr(rp), _ptr(ci), where), "atos_csr_create_part")
        g = CSR._wrap(h, n_global, int(ci.numel()), self.device, self.nranks)
        g.n_local = v_end - v_begin
        g.v_begin, g.v_end = v_begin, v_end
        g._comm_ref = self
        return g

    def gather(self, n_global: int, slice_: torch.Tensor, out: torch.Tensor | None = None):
        """atos_comm_gather: every rank's output slice -> one n_global array on rank 0 (None elsewhere)."""
        lib = _lib.load()
        if self.rank == 0 and out is None:
            out = torch.empty(n_global, dtype=slice_.dtype, device=slice_.device)
        stream = torch.cuda.current_stream(slice_.device)
        _lib.check(lib.atos_comm_gather(self._h, n_global, _ptr(slice_), slice_.element_size(),
                                        _ptr(out) if out is not None else None, ctypes.c_void_p(stream.cuda_stream)),
                   "atos_comm_gather")
        return out

    def close(self):
        if getattr(self, "_h", None) is not None:
            _lib.load().atos_comm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
