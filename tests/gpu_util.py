"""Helpers for the -m gpu parity tests (test infrastructure)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

NF = 24


def need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def to_dev(u_host, stride):
    """[nf, n] numpy -> [nf, stride] cuda float64 (zero padded)."""
    nf, n = u_host.shape
    t = torch.zeros((nf, stride), dtype=torch.float64, device="cuda")
    t[:, :n] = torch.from_numpy(np.ascontiguousarray(u_host))
    return t


def field_errors(gpu, ora):
    """Max-abs-relative error per field (DESIGN.md §Parity metric):
    err_f = max|gpu - ora| / max|ora_f|; for an identically-zero oracle field
    the error is max|gpu_f| / max_f' max|ora_f'| (compared against 1e-14)."""
    gpu = np.asarray(gpu, dtype=np.float64).reshape(gpu.shape[0], -1)
    ora = np.asarray(ora, dtype=np.float64).reshape(ora.shape[0], -1)
    scale_all = max(np.max(np.abs(ora)), 1e-300)
    out, zero = [], []
    for f in range(ora.shape[0]):
        s = np.max(np.abs(ora[f]))
        d = np.max(np.abs(gpu[f] - ora[f])) if ora.shape[1] else 0.0
        out.append(d / s if s > 0 else d / scale_all)
        zero.append(s == 0)
    return np.array(out), np.array(zero)


def assert_parity(gpu, ora, tol, what="", zero_tol=1e-14):
    e, zero = field_errors(gpu, ora)
    assert np.all(np.isfinite(np.asarray(gpu))), f"{what}: non-finite GPU values"
    bad = np.nonzero(np.where(zero, e > zero_tol, e > tol))[0]
    assert len(bad) == 0, f"{what}: fields {bad.tolist()} errors {e[bad]} (tol {tol:.1e}); all {e}"
    return e
