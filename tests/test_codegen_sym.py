"""The code generators' symbolic algebra (codegen/bssn_sym.py, written from
PAPER.md eqs 1-19 independently of oracle/) equals the oracle's algebra (which
tests/test_oracle_bssn.py pins to closed forms) on random inputs, and the
generated CUDA file is current (regenerating it gives the committed text)."""
import os

import numpy as np
import sympy as sp

from paper_conf_sc_fernandonhzsgb22_b200.codegen import bssn_sym, gen
from oracle import bssn

from .codegen_util import oracle_rhs, random_inputs, relerr


def test_symbolic_algebra_matches_oracle():
    exprs, syms, prm = bssn_sym.rhs_exprs()
    x = random_inputs(64, seed=7)
    p = bssn.Params(eta=1.7, lambda_f0=0.8, lambda_f1=0.3, chi_floor=0.6)
    args = list(syms) + [prm["eta"], prm["lambda_f0"], prm["lambda_f1"], prm["chi_e"]]
    f = sp.lambdify(args, exprs, modules="numpy", cse=True)
    chi_e = np.maximum(x[1], p.chi_floor)          # some chi below the floor: R13 exercised
    got = np.array([np.broadcast_to(v, (64,)) for v in
                    f(*x, p.eta, p.lambda_f0, p.lambda_f1, chi_e)])
    want = oracle_rhs(x, p)
    assert (x[1] < p.chi_floor).any()
    err = relerr(got, want)
    assert err.max() < 1e-12, err


def test_generated_file_is_current(tmp_path):
    with open(gen.OUT) as fh:
        committed = fh.read()
    out = tmp_path / "rhs_alg.cu"
    gen.main(str(out))
    assert out.read_text() == committed, "csrc/gen/rhs_alg.cu differs from the generator's output"
