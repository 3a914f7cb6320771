"""CPU-only checks of the C-ABI boundary: the library loads, exports every
symbol include/graffix.h declares, and fails loudly (no CPU fallback) when no
CUDA device is present."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "graffix.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gx_[a-z_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_icpp_0001n20_b200 import build
    build.build()
    from paper_conf_icpp_0001n20_b200._binding import lib
    return lib()


def test_exports_every_declared_symbol(L):
    from paper_conf_icpp_0001n20_b200._binding import EXPORTED
    syms = header_symbols()
    assert len(syms) >= 20
    assert sorted(EXPORTED) == syms
    for s in syms:
        assert hasattr(L, s), s


def test_abi_and_defaults(L):
    from paper_conf_icpp_0001n20_b200._binding import GxKnobs, GxRunOpts
    assert L.gx_abi_version() == 1
    k = GxKnobs()
    assert L.gx_knobs_default(C.byref(k)) == 0
    assert k.struct_size == C.sizeof(GxKnobs)
    assert (k.coalesce, k.smem, k.degree_norm) == (0, 0, 0)          # exact mode
    assert k.chunk_k == 16 and abs(k.replicate_threshold - 0.6) < 1e-15  # P@25752
    assert abs(k.degree_target - 0.85) < 1e-15                          # P@55220
    o = GxRunOpts()
    assert L.gx_run_opts_default(C.byref(o)) == 0 and o.struct_size == C.sizeof(GxRunOpts)


def test_no_cpu_fallback(L):
    """Without a GPU, context creation must fail with GX_E_CUDA."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    h = C.c_void_p()
    st = L.gx_ctx_create(C.byref(h), 0, None)
    assert st == 4
    assert b"CUDA" in L.gx_last_error() or b"device" in L.gx_last_error()


def test_null_arguments_rejected(L):
    assert L.gx_ctx_create(None, 0, None) == 1
    assert L.gx_knobs_default(None) == 1
    assert L.gx_graph_upload_csr(None, None, 0, 0, None, None, None, 0) == 1


def test_binding_constants_match_header():
    """Every #define / enum value the binding mirrors equals the header's."""
    from paper_conf_icpp_0001n20_b200 import _binding as B
    src = open(os.path.join(ROOT, "include", "graffix.h")).read()
    defs = {k: int(v) for k, v in re.findall(r"#define\s+(GX_[A-Z0-9_]+)\s+(\d+)u?\b", src)}
    for k, v in re.findall(r"\b(GX_[A-Z0-9_]+)\s*=\s*(\d+)", src):
        defs.setdefault(k, int(v))
    checked = 0
    for name in dir(B):
        if name.startswith("GX_") and name in defs and isinstance(getattr(B, name), int):
            assert getattr(B, name) == defs[name], name
            checked += 1
    assert checked >= 15
    for flag in ("GX_PTRS_DEVICE", "GX_VALIDATE", "GX_CANONICAL", "GX_ASYNC_UPLOAD", "GX_DL_ASYNC"):
        assert flag in defs and hasattr(B, flag), flag
    flags = [defs[f] for f in ("GX_PTRS_DEVICE", "GX_VALIDATE", "GX_CANONICAL", "GX_ASYNC_UPLOAD", "GX_DL_ASYNC")]
    assert all(f & (f - 1) == 0 for f in flags) and len(set(flags)) == len(flags)   # distinct single bits
