"""Helpers for the -m gpu parity tests (call the product through the C ABI)."""
import numpy as np
import pytest


def require_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")


_CTX = None


def ctx():
    global _CTX
    require_gpu()
    if _CTX is None:
        from paper_conf_icpp_0001n20_b200 import Context
        _CTX = Context(0)
    return _CTX


def upload(raw, **kw):
    from paper_conf_icpp_0001n20_b200 import Graph
    return Graph.upload(ctx(), raw.row_ptr, raw.col, raw.w, **kw)
