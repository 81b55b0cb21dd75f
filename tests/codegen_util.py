"""Helpers for the code-generation study tests: random inputs in the 234-input
layout of codegen/bssn_sym.py and their conversion to the oracle's PointData
layout (test infrastructure: may import oracle/)."""
from types import SimpleNamespace

import numpy as np

from oracle import bssn

SYM = [(0, 0), (0, 1), (0, 2), (1, 1), (1, 2), (2, 2)]
SECOND = [0, 1, 6, 7, 8, 12, 13, 14, 15, 16, 17]


def random_inputs(n, seed):
    """[234, n]: values in a physical range (gt near delta, chi and alpha in
    [0.5, 1.5]), derivatives and KO terms uniform in [-0.5, 0.5]."""
    rng = np.random.default_rng(seed)
    x = rng.uniform(-0.5, 0.5, size=(234, n))
    x[0] = rng.uniform(0.5, 1.5, n)
    x[1] = rng.uniform(0.5, 1.5, n)
    for q, (i, j) in enumerate(SYM):
        x[12 + q] = (1.0 if i == j else 0.0) + rng.uniform(-0.15, 0.15, n)
    return x


def full(v6):
    out = np.empty((3, 3) + v6.shape[1:])
    for q, (i, j) in enumerate(SYM):
        out[i, j] = out[j, i] = v6[q]
    return out


def to_pointdata(x):
    """234-input layout -> oracle.bssn.PointData-like namespace + KO sums [24, n]."""
    d = SimpleNamespace()
    d.alpha, d.chi, d.K = x[0], x[1], x[2]
    d.Gt, d.beta, d.B = x[3:6], x[6:9], x[9:12]
    d.gt, d.At = full(x[12:18]), full(x[18:24])
    D1 = lambda f: x[24 + 3 * f: 27 + 3 * f]                          # [k, n]
    d.d_alpha, d.d_chi, d.d_K = D1(0), D1(1), D1(2)
    d.d_Gt = np.stack([D1(3 + i) for i in range(3)], axis=1)          # [k, i]
    d.d_beta = np.stack([D1(6 + i) for i in range(3)], axis=1)
    d.d_B = np.stack([D1(9 + i) for i in range(3)], axis=1)
    d.d_gt = np.stack([full(np.stack([D1(12 + q)[k] for q in range(6)])) for k in range(3)])
    d.d_At = np.stack([full(np.stack([D1(18 + q)[k] for q in range(6)])) for k in range(3)])
    DD = lambda f: full(x[96 + 6 * SECOND.index(f): 102 + 6 * SECOND.index(f)])   # [k, l, n]
    d.dd_alpha, d.dd_chi = DD(0), DD(1)
    d.dd_beta = np.stack([DD(6 + i) for i in range(3)], axis=2)       # [k, l, i]
    d.dd_gt = np.empty((3, 3, 3, 3) + x.shape[1:])
    for q, (i, j) in enumerate(SYM):
        d.dd_gt[:, :, i, j] = d.dd_gt[:, :, j, i] = DD(12 + q)
    ko = np.stack([x[162 + 3 * f] + x[163 + 3 * f] + x[164 + 3 * f] for f in range(24)])
    return d, ko


def oracle_rhs(x, prm=None):
    d, ko = to_pointdata(x)
    return bssn.algebra(d, prm or bssn.Params()) + ko


def relerr(got, want):
    scale = np.maximum(np.abs(want).max(axis=1), 1e-300)
    return np.abs(got - want).max(axis=1) / scale


def eval_cse(exprs, values):
    """Evaluate SymPy expressions numerically through their CSE (fast for the
    large generated algebras): values maps input symbols to numpy arrays."""
    import sympy as sp
    rep, red = sp.cse(exprs, optimizations=None, order="none")
    env = dict(values)
    for t, e in rep + [(None, r) for r in red]:
        fs = sorted(e.free_symbols, key=lambda s: s.name)
        v = sp.lambdify(fs, e, modules="numpy")(*[env[s] for s in fs])
        if t is None:
            env.setdefault("__out__", []).append(v)
        else:
            env[t] = v
    return env["__out__"]
