"""Helpers for the -m gpu parity tests (test infrastructure)."""
import numpy as np
import pytest
import torch


def require_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_fengwcz0d21_b200 import egemm
    egemm.load()  # raises if the library is missing: no silent fallback
    return egemm


def to_dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def to_host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def u16(t):
    return to_host(t).view(np.uint16)
