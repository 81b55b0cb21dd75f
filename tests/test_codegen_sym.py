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
    from .codegen_util import eval_cse
    chi_e = np.maximum(x[1], p.chi_floor)          # some chi below the floor: R13 exercised
    vals = {s_: x[k] for k, s_ in enumerate(syms)}
    vals.update({prm["eta"]: p.eta, prm["lambda_f0"]: p.lambda_f0, prm["lambda_f1"]: p.lambda_f1,
                 prm["chi_e"]: chi_e})
    got = np.array([np.broadcast_to(v, (64,)) for v in eval_cse(exprs, vals)])
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


def test_generated_psi4_file_is_current(tmp_path):
    with open(gen.OUT_PSI4) as fh:
        committed = fh.read()
    out = tmp_path / "psi4.cu"
    gen.gen_psi4(str(out))
    assert out.read_text() == committed, "csrc/gen/psi4.cu differs from the generator's output"


def test_symbolic_psi4_matches_oracle():
    """codegen/psi4_sym.py (written from the readings independently of
    oracle/psi4.py) equals the oracle's Psi_4 on random inputs and positions."""
    from paper_conf_sc_fernandonhzsgb22_b200.codegen import psi4_sym
    from oracle import psi4 as op4
    from .codegen_util import to_pointdata
    exprs, syms, prm, (px, py, pz) = psi4_sym.psi4_exprs()
    x = random_inputs(32, seed=12)
    rng = np.random.default_rng(4)
    xyz = rng.uniform(-3, 3, size=(3, 32))
    p = bssn.Params(chi_floor=0.6)
    from .codegen_util import eval_cse
    vals = {s_: x[k] for k, s_ in enumerate(syms)}
    vals.update({prm["eta"]: p.eta, prm["lambda_f0"]: p.lambda_f0, prm["lambda_f1"]: p.lambda_f1,
                 prm["chi_e"]: np.maximum(x[1], p.chi_floor), px: xyz[0], py: xyz[1], pz: xyz[2]})
    re, im = eval_cse(exprs, vals)
    d, _ = to_pointdata(x)
    want = op4.psi4_point(d, xyz, p)
    assert np.abs(re + 1j * im - want).max() < 1e-11 * np.abs(want).max()
