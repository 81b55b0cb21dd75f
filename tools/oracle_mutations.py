"""Mutation check of the oracle's pins (VERDICT r1 "What's weak" #1-2).

Each mutation below is a plausible transcription mistake in oracle/bssn.py or
oracle/constraints.py (a dropped term, a wrong sign, a transposed index, a
wrong weight).  For each one the repository is copied to a scratch directory,
the mutation applied, and the -m "not gpu" oracle pins run; a mutation that
no pin fails is a gap in the pins.  Output: one line per mutation,
KILLED/SURVIVED.  Usage: python tools/oracle_mutations.py [> profiles/...]
"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

B = "oracle/bssn.py"
C = "oracle/constraints.py"
MUTATIONS = [
    # eq (1)
    (B, 'out[F_ALPHA] = adv(F_ALPHA, d.d_alpha) - 2.0 * a * K', 'out[F_ALPHA] = - 2.0 * a * K', "eq1 drop advection"),
    (B, 'out[F_ALPHA] = adv(F_ALPHA, d.d_alpha) - 2.0 * a * K', 'out[F_ALPHA] = adv(F_ALPHA, d.d_alpha) + 2.0 * a * K', "eq1 sign of 2aK"),
    # eq (2)
    (B, 'adv(F_BETA + i, d.d_beta[:, i])', 'adv(F_BETA + i, d.d_beta[i, :])', "eq2 transposed self-advection"),
    (B, '+ 0.75 * f_alpha * d.B[i]', '+ 0.5 * f_alpha * d.B[i]', "eq2 3/4 -> 1/2"),
    # eq (3)
    (B, 'out[F_B + i] = (rhs_Gt[i] - prm.eta', 'out[F_B + i] = (- prm.eta', "eq3 drop d_t Gt"),
    (B, '- adv(F_GT + i, d.d_Gt[:, i]))', ')', "eq3 drop -beta.grad Gt"),
    (B, '+ adv(F_B + i, d.d_B[:, i])', '', "eq3 drop beta.grad B"),
    (B, 'adv(F_B + i, d.d_B[:, i])', 'adv(F_B + i, d.d_B[i, :])', "eq3 transposed beta.grad B"),
    # eq (4), Lie derivative
    (B, '- (2.0 / 3.0) * T * div_beta)', '- (0.0 / 3.0) * T * div_beta)', "eq10 weight 0"),
    (B, '+ np.einsum("ik...,jk...->ij...", T, d.d_beta)', '+ np.einsum("ik...,kj...->ij...", T, d.d_beta)', "eq10 transposed d beta"),
    (B, 'rhs_gt = lie(d.gt, d.d_gt) - 2.0 * a * d.At', 'rhs_gt = lie(d.gt, d.d_gt) + 2.0 * a * d.At', "eq4 sign of 2 a At"),
    # eq (5)
    (B, '(2.0 / 3.0) * d.chi * (a * K - div_beta)', '(2.0 / 3.0) * d.chi * (a * K + div_beta)', "eq5 sign div beta"),
    (B, 'out[F_CHI] = adv(F_CHI, d.d_chi) +', 'out[F_CHI] = 0.0 +', "eq5 drop advection"),
    # eq (6)
    (B, 'd.chi * tf(-G["DDa"] + a * G["Ric"])', 'd.chi * tf(G["DDa"] + a * G["Ric"])', "eq6 sign DDa"),
    (B, 'd.chi * tf(-G["DDa"] + a * G["Ric"])', 'd.chi * (-G["DDa"] + a * G["Ric"])', "eq6 drop trace-free"),
    (B, '+ a * (K * d.At - 2.0 * np.einsum("ik...,kj...->ij...", d.At, A_mix)))',
        '+ a * (K * d.At - 1.0 * np.einsum("ik...,kj...->ij...", d.At, A_mix)))', "eq6 2 AA -> 1 AA"),
    (B, 'return T - d.gt * tr / 3.0', 'return T - d.gt * tr / 2.0', "eq11 1/3 -> 1/2"),
    # eq (7)
    (B, 'out[F_K] = adv(F_K, d.d_K) - G["DDa_tr"]', 'out[F_K] = adv(F_K, d.d_K) + G["DDa_tr"]', "eq7 sign DDa_tr"),
    (B, '+ K * K / 3.0)', '+ K * K / 2.0)', "eq7 K^2/3 -> K^2/2"),
    # eq (8)
    (B, 'rhs_Gt = (np.einsum("jk...,jki...->i...", ginv, d.dd_beta)', 'rhs_Gt = (0.0', "eq8 drop laplacian beta"),
    (B, '+ np.einsum("ij...,j...->i...", ginv, dd_beta_div) / 3.0', '+ np.einsum("ij...,j...->i...", ginv, dd_beta_div) / 6.0', "eq8 1/3 -> 1/6"),
    (B, '+ np.stack([adv(F_GT + i, d.d_Gt[:, i]) for i in range(3)])', '+ np.stack([adv(F_GT + i, d.d_Gt[i, :]) for i in range(3)])', "eq8 transposed beta.grad Gt"),
    (B, '- np.einsum("j...,ji...->i...", CalGt, d.d_beta)', '+ np.einsum("j...,ji...->i...", CalGt, d.d_beta)', "eq8 sign CalGt d beta"),
    (B, '+ (2.0 / 3.0) * CalGt * div_beta', '- (2.0 / 3.0) * CalGt * div_beta', "eq8 sign CalGt div beta"),
    (B, '- 2.0 * np.einsum("ij...,j...->i...", A_up, d.d_alpha)', '+ 2.0 * np.einsum("ij...,j...->i...", A_up, d.d_alpha)', "eq8 sign At d alpha"),
    (B, '+ 2.0 * a * (np.einsum("ijk...,jk...->i...", Gam, A_up)', '+ 2.0 * a * (0.0', "eq8 drop Gam At"),
    (B, '- 1.5 / chi * np.einsum("ij...,j...->i...", A_up, d.d_chi)', '- 1.0 / chi * np.einsum("ij...,j...->i...", A_up, d.d_chi)', "eq8 3/2 -> 1"),
    (B, '- (2.0 / 3.0) * np.einsum("ij...,j...->i...", ginv, d.d_K)))', '- (1.0 / 3.0) * np.einsum("ij...,j...->i...", ginv, d.d_K)))', "eq8 2/3 -> 1/3"),
    # geometry
    (B, 'Gam = np.einsum("kl...,lij...->kij...", ginv, C)', 'Gam = np.einsum("kl...,ijl...->kij...", ginv, C)', "eq12 index"),
    (B, "- np.einsum(\"ij...,kl...,l...->kij...\", d.gt, ginv, d.d_chi)) / (2.0 * chi)",
        "+ np.einsum(\"ij...,kl...,l...->kij...\", d.gt, ginv, d.d_chi)) / (2.0 * chi)", "eq13 sign"),
    (B, 'Rt = (-0.5 * np.einsum', 'Rt = (0.5 * np.einsum', "eq17 printed +1/2"),
    (B, '+ np.einsum("lm...,kim...,klj...->ij...", ginv, Gam, Gl))', ')', "eq17 drop third GG term"),
    (B, '- np.einsum("i...,j...->ij...", d.d_chi, d.d_chi) / (4.0 * chi * chi)', '', "eq18 drop dchi dchi"),
    (B, '- np.einsum("m...,m...->...", CalGt, d.d_chi)))', '))', "eq19 drop CalGt dchi"),
    (B, 'DDa_tr = d.chi * np.einsum', 'DDa_tr = np.einsum', "eq14 drop chi"),
    # constraints
    (C, '+ (2.0 / 3.0) * d.K * d.K - np.einsum', '+ (1.0 / 3.0) * d.K * d.K - np.einsum', "H 2/3 -> 1/3"),
    # (d_j At^ij -> d_i At^ij is an equivalent mutant: At^ij is symmetric)
    (C, 'M = (np.einsum("jij...->i...", d_Aup)', 'M = (np.einsum("ijj...->i...", d_Aup)', "M divergence -> gradient of trace"),
    (C, '- 1.5 / chi * np.einsum("ij...,j...->i...", A_up, d.d_chi))', ')', "M drop chi term"),
    (C, 'Gc = d.Gt - G["CalGt"]', 'Gc = d.Gt + G["CalGt"]', "G sign"),
]

TESTS = ["tests/test_oracle_bssn.py", "tests/test_oracle_boundary.py"]


def main():
    tmp = tempfile.mkdtemp(prefix="dgr_mut_")
    src = os.path.join(tmp, "repo")
    shutil.copytree(ROOT, src, ignore=shutil.ignore_patterns(".git", "gpurun_out", "profiles", "*.so"))
    survived = 0
    for f, old, new, what in MUTATIONS:
        path = os.path.join(src, f)
        orig = open(path).read()
        if orig.count(old) != 1:
            print(f"BADPATTERN {what}: {orig.count(old)} matches", flush=True)
            continue
        open(path, "w").write(orig.replace(old, new))
        r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider"] + TESTS,
                           cwd=src, capture_output=True, text=True)
        open(path, "w").write(orig)
        fails = [l.split("::")[1].split(" ")[0] for l in r.stdout.splitlines() if l.startswith("FAILED")]
        if r.returncode == 0:
            survived += 1
            print(f"SURVIVED {what}", flush=True)
        else:
            print(f"KILLED   {what}  by {','.join(fails) or r.stdout.strip().splitlines()[-1]}", flush=True)
    print(f"{len(MUTATIONS)} mutations, {survived} survived")
    shutil.rmtree(tmp, ignore_errors=True)


if __name__ == "__main__":
    main()
