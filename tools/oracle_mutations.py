"""Mutation check of the oracle pins.

Each mutant is one plausible mistake in oracle/pf_oracle.c (a dropped term, a
wrong sign, factor, index or operand).  A mutant is compiled from a copy of
the source in a temporary directory (the repo file is never touched; the
oracle binding picks the copy up through PF_ORACLE_SRC / PF_ORACLE_LIB) and
the pins are run against it in a subprocess: a pin failing = the mutant is
CAUGHT.  `catch` names the pins expected to catch each mutant (the quick
selection used by tests/test_oracle_mutations.py); `python
tools/oracle_mutations.py --full` runs the whole pin file per mutant instead.

Equivalent mutants (no observable change) are listed with catch=None and the
reason.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "pf_oracle.c")
PINS = "tests/test_oracle_pins.py"

# (original text, mutated text, pins expected to catch it | None = equivalent)
MUTANTS = [
    ("16.0 / (PI_D * PI_D)", "8.0 / (PI_D * PI_D)", ["test_p4_sine_profile_stationary"]),
    ("(PI_D * p->eps / 4.0)", "(PI_D * p->eps / 2.0)", ["test_antitrapping_1d_closed_form"]),
    ("(4.0 * p->dx);\n    }", "(2.0 * p->dx);\n    }", ["test_antitrapping_diagonal_front"]),
    ("xs[a] = ph[a] + f * (-r[a] + lam + xi[a]);", "xs[a] = ph[a] + f * (r[a] - lam + xi[a]);",
     ["test_p4_sine_profile_stationary", "test_p15_energy_decay"]),
    ("xs[a] = ph[a] + f * (-r[a] + lam + xi[a]);", "xs[a] = ph[a] + f * (-r[a] + lam - xi[a]);",
     ["test_xi_enters_the_euler_step"]),
    ("return 6.0 * x * (1.0 - x);", "return 3.0 * x * (1.0 - x);", ["test_p6_front_velocity"]),
    ("Q[i] += h * cT[i] * dTdt;", "Q[i] += h * cT[i];", ["test_p9_temperature_Q_term"]),
    ("Mf[i][j] += g_of(pb[a]) * s;", "Mf[i][j] += h_of(pb[a]) * s;", ["test_mobility_face_interpolation"]),
    ("s += p->D[a][i][k] * chi[k][j];", "s += chi[i][k] * p->D[a][k][j];", ["test_p8_product_order_D_chi"]),
    ("(gr[a][d] / nrm_a);", "(gr[L][d] / nrm_l);", ["test_antitrapping_1d_closed_form"]),
    ("S[i] += c[i] * dh * dtphi;", "S[i] -= c[i] * dh * dtphi;", ["test_p10_solute_flux_identity"]),
    ("(chi[1][1] * rhs[0] - chi[0][1] * rhs[1]) / det", "(chi[1][1] * rhs[0] - chi[1][0] * rhs[1]) / det",
     None),  # equivalent: chi = -(A + A^T) is symmetric by construction [A6]
    ("s += p->gamma[a][b] * pb[b] * (pb[b] * dd[a] - pb[a] * dd[b]);",
     "s += p->gamma[a][b] * pb[a] * (pb[b] * dd[a] - pb[a] * dd[b]);", ["test_p5_third_phase_bound"]),
    ("(double)z + (d == 2 ? 0.5 : 0.0)", "(double)z", ["test_mobility_temperature_at_faces"]),
    ("double lam = rs / (double)N;", "double lam = rs / (double)(N-1);", ["test_p2_simplex_invariants"]),
    ("om += gamma3_of(p, a, b, d) * ph[b] * ph[d];", "om += 0.5*gamma3_of(p, a, b, d) * ph[b] * ph[d];",
     ["test_p5_third_phase_bound", "test_p7_sympy_variational_derivative"]),
    ("r[a] = p->eps * (dadphi - div[a]) + om / p->eps + dpsi;",
     "r[a] = p->eps * (dadphi + div[a]) + om / p->eps + dpsi;", ["test_p4_sine_profile_stationary"]),
    ("double tau = den != 0.0 ? num / den : tsum / (double)npair;",
     "double tau = den != 0.0 ? num / den / 2 : tsum / (double)npair;", ["test_p6_front_velocity"]),
    # reading A5: the tau interpolation itself
    ("double tau = den != 0.0 ? num / den : tsum / (double)npair;",
     "double tau = tsum / (double)npair;", ["test_a5_tau_binary_front_speed"]),
    ("num += p->tau[a][b] * ph[a] * ph[b];", "num += p->tau[a][b] * (ph[a] + ph[b]);",
     ["test_a5_tau_limits_in_cells"]),
    ("double tau = den != 0.0 ? num / den : tsum / (double)npair;",
     "double tau = den != 0.0 ? num / den : p->tau[0][1];", ["test_a5_tau_limits_in_cells"]),
    ("c[i] = -s - B[i];", "c[i] = -s + B[i];", ["test_p10_solute_flux_identity"]),
    ("out[i] = -s - p->B1[a][i];", "out[i] = s - p->B1[a][i];", ["test_p9_temperature_Q_term"]),
    ("double dTdt = -p->G * p->v;", "double dTdt = p->G * p->v;", ["test_p9_temperature_Q_term"]),
    ("for (int d = 0; d < 3; ++d) dot += (ph[a] * g[b][d] - ph[b] * g[a][d]) * g[b][d];",
     "for (int d = 0; d < 3; ++d) dot += (ph[a] * g[b][d] - ph[b] * g[a][d]) * g[a][d];",
     ["test_p7_sympy_variational_derivative"]),
    ("if (!(pb[a] > 0.0 && pb[L] > 0.0 && na2 > 0.0 && nl2 > 0.0)) continue;",
     "if (!(pb[a] > 0.0 && pb[L] > 0.0 && na2 > 0.0 && nl2 > 0.0)) continue; if (a==0) continue;",
     ["test_antitrapping_1d_closed_form"]),
    ("dtp[a] = ((rd(o, F_PHI_DST, a, x, y, z) - vp) + (rd(o, F_PHI_DST, a, qx, qy, qz) - vq)) / (2.0 * p->dt);",
     "dtp[a] = ((rd(o, F_PHI_DST, a, x, y, z) - vp) + (rd(o, F_PHI_DST, a, qx, qy, qz) - vq)) / (1.0 * p->dt);",
     ["test_antitrapping_1d_closed_form"]),
    # reading A15: the Dirichlet-mu ghost
    ("val = o->p.mu_inf[c];", "val = 0.0;", ["test_a15_dirichlet_mu_top"]),
    ("} else if (bc == OR_BC_DIRICHLET_MU && is_mu) {", "} else if (bc == OR_BC_DIRICHLET_MU && !is_mu) {",
     ["test_a15_dirichlet_mu_top"]),
    ("int src_neu = side ? n[d] - 1 : 0;", "int src_neu = side ? n[d] - 2 : 1;", ["test_mobility_face_interpolation"]),
    # reading B6 (P2 anisotropy)
    ("for (int j = 0; j < 3; ++j) out[j] = R[0][j] * gp[0] + R[1][j] * gp[1] + R[2][j] * gp[2];",
     "for (int j = 0; j < 3; ++j) out[j] = R[j][0] * gp[0] + R[j][1] * gp[1] + R[j][2] * gp[2];",
     ["tests/test_oracle_p2.py::test_p2_lattice_rotation_covariance"]),
    ("gp[i] = 2.0 * A * dA * n2 + 2.0 * A * A * v[i];", "gp[i] = 2.0 * A * A * v[i];",
     ["tests/test_oracle_p2.py::test_p2_sympy_variational_derivative"]),
    ("double A = 1.0 - delta * (3.0 - 4.0 * s4 / (n2 * n2));", "double A = 1.0 + delta * (3.0 - 4.0 * s4 / (n2 * n2));",
     ["tests/test_oracle_p2.py::test_p2_planar_profile_width"]),
    ("s += p->gamma[a][b] * (-pb[b]) * gf[d];", "s += p->gamma[a][b] * (-pb[a]) * gf[d];",
     ["tests/test_oracle_p2.py::test_p2_sympy_variational_derivative"]),
    ("if (e == d) { G[b][e] = dd[b]; continue; }", "if (1) { G[b][e] = e == d ? dd[b] : 0.0; continue; }",
     ["tests/test_oracle_p2.py::test_p2_sympy_variational_derivative", "tests/test_oracle_p2.py::test_p2_table1_footprint"]),
    # reading A16: window inflow
    ("mu[idx(o, i, x, y, z)] = z + k < nz ? mu[idx(o, i, x, y, z + k)] : o->p.mu_inf[i];",
     "mu[idx(o, i, x, y, z)] = z + k < nz ? mu[idx(o, i, x, y, z + k)] : 0.0;", ["test_window_shift_semantics"]),
]


def run_mutant(i: int, full: bool = False, timeout: float = 600.0):
    """Build mutant i from a temporary copy and run its pins.  Returns
    (i, caught: bool | None, first failing pin)."""
    a, b, catch = MUTANTS[i]
    orig = open(SRC).read()
    assert orig.count(a) >= 1, f"mutant {i}: original text not found: {a!r}"
    with tempfile.TemporaryDirectory(prefix=f"orm{i}_") as td:
        src = os.path.join(td, "pf_oracle.c")
        open(src, "w").write(orig.replace(a, b, 1))
        env = dict(os.environ, PF_ORACLE_SRC=src, PF_ORACLE_LIB=os.path.join(td, "libpf_oracle.so"),
                   OMP_NUM_THREADS="1")
        sel = ([PINS, "tests/test_oracle_p2.py"] if (full or catch is None)
               else [t if "::" in t else f"{PINS}::{t}" for t in catch])
        r = subprocess.run([sys.executable, "-m", "pytest", *sel, "-q", "-x", "-p", "no:cacheprovider"],
                           capture_output=True, text=True, cwd=ROOT, env=env, timeout=timeout)
    fails = [ln.split()[1] for ln in r.stdout.splitlines() if ln.startswith("FAILED")]
    return i, bool(fails), (fails[0] if fails else "")  # a build error is not a catch


def main(argv):
    full = "--full" in argv
    workers = min(8, os.cpu_count() or 1)
    with cf.ThreadPoolExecutor(workers) as ex:
        res = sorted(ex.map(lambda i: run_mutant(i, full), range(len(MUTANTS))))
    n_caught = 0
    for i, caught, first in res:
        a, b, catch = MUTANTS[i]
        tag = "CAUGHT" if caught else ("EQUIV " if catch is None else "MISSED")
        n_caught += bool(caught)
        print(f"{tag} {i:2d} {b[:70]!r} {first}")
    print(f"{n_caught} of {len(MUTANTS)} caught "
          f"({sum(c is None for _, _, c in MUTANTS)} listed as equivalent)")


if __name__ == "__main__":
    main(sys.argv[1:])
