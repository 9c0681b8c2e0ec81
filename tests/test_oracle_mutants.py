"""Mutation test of the oracle's pins: each mutant is a plausible mistake in
oracle/idg_oracle.c -- a flipped sign, a dropped term, a transposed or mis-indexed operand, an
off-by-one -- compiled on its own and run against the pin suites (tests/test_oracle_pins.py,
tests/test_oracle_plan.py).  Every mutant must fail at least one pin: the pins fix the oracle, not
the other way round."""
import os
import subprocess
import sys
import tempfile
from concurrent.futures import ThreadPoolExecutor

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "idg_oracle.c")

# (name, original text, mutated text); each original occurs exactly once in idg_oracle.c
MUTANTS = [
    ("gridder phasor conjugated (e^{-i phi})", "double complex phasor = cos(phi) + I * sin(phi);",
     "double complex phasor = cos(phi) - I * sin(phi);"),
    ("degridder phase sign (alpha = +f.g)", "double alpha = -or_phase(", "double alpha = or_phase("),
    ("w-term dropped", "(v - v0) * m + (w - w0) * n)", "(v - v0) * m)"),
    ("n sign (north-star n - 1 form)", "*n = 1.0 - sqrt(1.0 - (*l) * (*l) - (*m) * (*m));",
     "*n = sqrt(1.0 - (*l) * (*l) - (*m) * (*m)) - 1.0;"),
    ("l and m transposed", "*l = (double)(x - Ns / 2) * L / (double)Ns;\n    *m = (double)(y - Ns / 2) * L / (double)Ns;",
     "*l = (double)(y - Ns / 2) * L / (double)Ns;\n    *m = (double)(x - Ns / 2) * L / (double)Ns;"),
    ("half-pixel shift in l", "*l = (double)(x - Ns / 2) * L", "*l = ((double)(x - Ns / 2) + 0.5) * L"),
    ("subgrid centre u0 off by one cell", "double u0 = (double)(it->x + Ns / 2 - N / 2) / L;",
     "double u0 = (double)(it->x + Ns / 2 - N / 2 + 1) / L;"),
    ("u and v columns swapped", "double u = (double)p[0] * freq", "double u = (double)p[1] * freq"),
    ("W-plane centre ignored (w0 = w_offset)", "double w0 = or_w0(P, it->z);", "double w0 = P->w_offset;"),
    ("gridder DFT sign", "oracle_centred_dft(Ns, -1, plane,", "oracle_centred_dft(Ns, +1, plane,"),
    ("degridder DFT sign", "oracle_centred_dft(Ns, +1, subgrid_in", "oracle_centred_dft(Ns, -1, subgrid_in"),
    ("DFT not centred in k", "int64_t e = (int64_t)(ky - h) * (y - h)", "int64_t e = (int64_t)(ky) * (y - h)"),
    ("gridder A_p not conjugated", "or_mat_adjoint(Ap, ApH);", "for (int k = 0; k < 4; k++) ApH[k] = Ap[k];"),
    ("degridder A_q not conjugated", "or_mat_adjoint(Aq, AqH);", "for (int k = 0; k < 4; k++) AqH[k] = Aq[k];"),
    ("adjoint without transpose", "AH[1] = conj(A[2]);\n    AH[2] = conj(A[1]);", "AH[1] = conj(A[1]);\n    AH[2] = conj(A[2]);"),
    ("2x2 product mis-indexed", "C[1] = A[0] * B[1] + A[1] * B[3];", "C[1] = A[0] * B[1] + A[1] * B[2];"),
    ("gridder stations swapped", "or_mat_mul(ApH, &S[(y * Ns + x) * 4], tmp);\n            or_mat_mul(tmp, Aq, res);",
     "or_mat_mul(ApH, &S[(y * Ns + x) * 4], tmp);\n            or_mat_mul(tmp, Ap, res);"),
    ("gridder taper skipped", "or_mat_mul(tmp, Aq, res);\n            double s = (double)taper[y * Ns + x];",
     "or_mat_mul(tmp, Aq, res);\n            double s = 1.0;"),
    ("degridder taper skipped", "or_mat_mul(tmp, AqH, res);\n            double s = (double)taper[y * Ns + x];",
     "or_mat_mul(tmp, AqH, res);\n            double s = 1.0;"),
    ("gridder taper transposed", "or_mat_mul(tmp, Aq, res);\n            double s = (double)taper[y * Ns + x];",
     "or_mat_mul(tmp, Aq, res);\n            double s = (double)taper[x * Ns + y];"),
    ("degridder taper transposed", "or_mat_mul(tmp, AqH, res);\n            double s = (double)taper[y * Ns + x];",
     "or_mat_mul(tmp, AqH, res);\n            double s = (double)taper[x * Ns + y];"),
    ("adder one row low", "grid[(((int64_t)it->z * 4 + pol) * N + it->y + ky) * N + it->x + kx] +=",
     "grid[(((int64_t)it->z * 4 + pol) * N + it->y + ky + 1) * N + it->x + kx] +="),
    ("splitter transposed", "int64_t g = (((int64_t)it->z * 4 + pol) * N + it->y + ky) * N + it->x + kx;",
     "int64_t g = (((int64_t)it->z * 4 + pol) * N + it->x + kx) * N + it->y + ky;"),
    ("plan: kernel support ignored", "return (bb->umax - bb->umin) + (double)K <= (double)Ns &&",
     "return (bb->umax - bb->umin) <= (double)Ns &&"),
    ("plan: T~max off by one", "while (t + nt < T && t + nt < slot_end && nt < Tmax) {",
     "while (t + nt < T && t + nt < slot_end && nt <= Tmax) {"),
    ("plan: A-term slots ignored", "while (t + nt < T && t + nt < slot_end && nt < Tmax) {",
     "while (t + nt < T && nt < Tmax) {"),
    ("plan: position rounded down", "int x = (int)floor((bb.umin + bb.umax) / 2.0 + (double)(N / 2) + 0.5) - Ns / 2;",
     "int x = (int)floor((bb.umin + bb.umax) / 2.0 + (double)(N / 2)) - Ns / 2;"),
    ("plan: drops not counted", "dropped += (int64_t)nt * (c1 - c0);", "(void)0;"),
    ("plan: W-plane break ignored", "if (or_w_plane(P, uvw, T, b, t + nt, nu_ref) != z) break;", "(void)0;"),
]

PIN_SUITES = ["tests/test_oracle_pins.py", "tests/test_oracle_plan.py"]


def _run_mutant(tmp, idx, old, new):
    src = open(SRC).read()
    assert src.count(old) == 1, f"mutant {idx}: pattern occurs {src.count(old)} times"
    path_c = os.path.join(tmp, f"m{idx}.c")
    path_so = os.path.join(tmp, f"m{idx}.so")
    open(path_c, "w").write(src.replace(old, new))
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-D_GNU_SOURCE", "-fopenmp", "-ffp-contract=off",
                           "-fPIC", "-shared", "-o", path_so, path_c, "-lm"])
    env = dict(os.environ, IDG_ORACLE_LIB=path_so, OMP_NUM_THREADS="2")
    r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-rf", "-p", "no:cacheprovider", "-m",
                        "not gpu", *PIN_SUITES], cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    killer = next((ln.split()[1] for ln in r.stdout.splitlines() if ln.startswith("FAILED ")), None)
    return r.returncode, killer, r.stdout[-800:]


def test_unmutated_oracle_passes_the_pins():
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider", "-m", "not gpu",
                        *PIN_SUITES], cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:]


def test_every_mutant_is_killed_by_a_pin():
    with tempfile.TemporaryDirectory() as tmp, ThreadPoolExecutor(max_workers=8) as ex:
        futs = [ex.submit(_run_mutant, tmp, i, old, new) for i, (_, old, new) in enumerate(MUTANTS)]
        results = [f.result() for f in futs]
    # killed = pytest exit code 1 (tests failed) with a named failing pin; a crash, a collection error or
    # a passing run is not a kill
    survivors = [f"{name}: rc={rc} {out}" for (name, _, _), (rc, killer, out) in zip(MUTANTS, results)
                 if rc != 1 or killer is None]
    assert not survivors, "mutants not killed by a pin:\n" + "\n".join(survivors)
    for (name, _, _), (_, killer, _) in zip(MUTANTS, results):
        print(f"{name:45s} killed by {killer}")
