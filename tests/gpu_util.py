"""Helpers for the -m gpu parity tests (CUDA path through the C ABI vs the oracle)."""
import numpy as np
import pytest
import torch

DEV = torch.device("cuda:0")


def to_dev(a, dtype=torch.float64):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV, dtype=dtype)


def to_host(t):
    torch.cuda.synchronize()
    return t.detach().cpu().numpy().astype(np.float64)


def assert_abs_close(got, ref, bound, rtol, what=""):
    """DESIGN.md R14: |gpu - oracle| <= rtol * S componentwise, S = abs-value evaluation."""
    got = np.asarray(got)
    assert got.shape == ref.shape, (got.shape, ref.shape)
    assert np.all(np.isfinite(got)), f"{what}: non-finite output (unwritten / poisoned?)"
    err = np.abs(got - ref)
    lim = rtol * np.asarray(bound) + 1e-300
    bad = err > lim
    if bad.any():
        i = np.argmax(err / lim)
        pytest.fail(f"{what}: {bad.sum()} of {bad.size} outside tolerance; worst idx {np.unravel_index(i, err.shape)}"
                    f" err {err.flat[i]:.3e} bound {lim.flat[i]:.3e}")


def poisoned_like(t):
    return torch.full_like(t, float("nan"))
