"""C-ABI boundary tests that need no GPU: the library loads, exports every
symbol include/atos.h declares, the cfg/stats struct layouts agree with the
binding, pure host functions work, and device calls fail loudly (no CPU
fallback) when there is no GPU."""
import ctypes
import os
import re

import pytest
import torch

from paper_conf_icpp_chenbpbyo22_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "atos.h")).read()
    return sorted(set(re.findall(r"ATOS_API\s+[\w\s\*]+?\b(atos_\w+)\s*\(", src)))


def test_header_lists_match_binding():
    assert header_symbols() == sorted(_lib.EXPORTS)


def test_library_exports_every_symbol():
    lib = _lib.load()
    for s in header_symbols():
        assert hasattr(lib, s), s
    assert lib.atos_version() == 1


def test_nm_dynamic_symbols():
    import subprocess
    _lib.load()
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True).stdout
    syms = set(re.findall(r"\b(atos_\w+)\b", out))
    assert set(header_symbols()) <= syms
    # hidden visibility: nothing but the ABI leaks from our own code
    assert not any(s.startswith("_ZN4atos") for s in out.split())


def test_cfg_layout_and_defaults():
    cfg = _lib.default_cfg()
    assert cfg.struct_size == ctypes.sizeof(_lib.Cfg)
    assert cfg.persistent == 1 and cfg.dedupe == 1 and cfg.out_where == _lib.MEM_DEVICE
    assert ctypes.sizeof(_lib.Stats) == 10 * 8 + 8 * 2
    # barrier_free took the last reserved int: the struct keeps its size, the field is the last int
    assert cfg.barrier_free == 0
    assert _lib.Cfg.barrier_free.offset == _lib.Cfg.engine_variant.offset + 4


def test_partition_range():
    import paper_conf_icpp_chenbpbyo22_b200 as atos
    n, P = 1000003, 8
    spans = [atos.partition_range(n, P, p) for p in range(P)]
    assert spans[0][0] == 0 and spans[-1][1] == n
    for (a, b), (c, d) in zip(spans, spans[1:]):
        assert b == c and a <= b
    with pytest.raises(RuntimeError):
        atos.partition_range(10, 0, 0)


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU failure path")
def test_no_gpu_fails_loudly():
    import paper_conf_icpp_chenbpbyo22_b200 as atos
    rp = torch.tensor([0, 1, 2], dtype=torch.int64)
    ci = torch.tensor([1, 0], dtype=torch.int32)
    with pytest.raises(RuntimeError, match="ATOS_ERR_CUDA"):
        atos.CSR(rp, ci)


def test_last_error_and_invalid_args():
    lib = _lib.load()
    h = ctypes.c_void_p()
    rc = lib.atos_csr_create(ctypes.byref(h), -1, 0, None, None, 0, 0, 1)
    assert rc == -1
    assert b"invalid" in lib.atos_last_error()
