"""Pins of the CPU oracle against what the paper and the mathematics fix
(SURVEY §8(c)-C.3 / DESIGN.md §5).  CPU only (-m "not gpu").

Each test names the pin it implements and the passage it follows.  None of
them re-types the oracle's formulas: they check closed forms, invariants,
brute force, an independent symbolic derivation (sympy) or the paper's
Table 1.
"""
import itertools
import json
import os

import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
from tests._pins_common import (BC_PERIODIC, BC_X_NEUMANN, front_position, simple_params,
                                sine_profile)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# --------------------------------------------------------------------------
# P14: Table 1 per-cell loads / stores reproduced exactly by
# the oracle's stencil reading (A8-A10).
# --------------------------------------------------------------------------
def test_p14_table1_footprint(oracle_mod):
    gold = json.load(open(os.path.join(GOLDEN, "table1_p1.json")))
    o = oracle_mod.Oracle((6, 6, 6), I.params_c4())
    phi, mu = I.ic_random((6, 6, 6))
    o.init(phi, mu)
    for k in gold["loads"]:
        loads, stores = o.footprint(k, (2, 3, 2))
        assert loads == gold["loads"][k], (k, loads)
        assert stores == gold["stores"][k], (k, stores)


# --------------------------------------------------------------------------
# P1: Gibbs-simplex projection [A14] == brute force over all faces of the
# simplex, plus the KKT conditions.
# --------------------------------------------------------------------------
def _project_brute(x):
    """Nearest point of the simplex by enumerating every face (active set)."""
    N = len(x)
    best, bd = None, np.inf
    for r in range(1, N + 1):
        for S in itertools.combinations(range(N), r):
            S = list(S)
            y = np.zeros(N)
            y[S] = x[S] - (x[S].sum() - 1.0) / r
            if np.all(y[S] >= -1e-14):
                d = np.sum((y - x) ** 2)
                if d < bd:
                    bd, best = d, y
    return best


@pytest.mark.parametrize("N", [2, 3, 4])
def test_p1_projection_bruteforce_and_kkt(oracle_mod, N):
    rng = np.random.default_rng(N)
    for trial in range(3000):
        x = rng.normal(0.3, 0.6, size=N) if trial % 2 else rng.uniform(-0.5, 1.5, size=N)
        y = oracle_mod.project_simplex(x)
        assert np.all(y >= 0.0)
        assert abs(y.sum() - 1.0) <= 4e-16 * N
        np.testing.assert_allclose(y, _project_brute(x), atol=2e-15)
        # KKT: x - y = theta * 1 - lambda, lambda >= 0, lambda_a y_a = 0
        theta = np.mean((x - y)[y > 0])
        lam = theta - (x - y)
        assert np.all(lam[y > 0] == pytest.approx(0.0, abs=2e-15))
        assert np.all(lam[y == 0] >= -2e-15)


def test_p1_projection_pure_stays_exact(oracle_mod):
    """C.6.2: with rho = 1, theta = u1 - 1 and phi = x - theta == 1 exactly."""
    for d in [1e-3, 0.2, 0.7]:
        y = oracle_mod.project_simplex(np.array([-d, 1.0 + d / 3, -2 * d, -0.5 * d]))
        assert y.tolist() == [0.0, 1.0, 0.0, 0.0]


# --------------------------------------------------------------------------
# P2: sum phi = 1 and phi >= 0 after every step; without the projection the
# Lagrange multiplier alone keeps sum phi = 1 (eq. 7) [A1, A3].
# --------------------------------------------------------------------------
@pytest.mark.parametrize("ic", ["R", "V"])
def test_p2_simplex_invariants(oracle_mod, ic):
    P = I.params_stress()
    shape = (8, 10, 12)
    phi, mu = I.make_ic(ic, shape, seed=2)
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    for _ in range(5):
        o.step(1)
        p, _ = o.download()
        assert np.abs(p.sum(0) - 1.0).max() <= 8 * 2.2e-16
        assert p.min() >= 0.0
    Pn = dict(P, projection=0)
    o = oracle_mod.Oracle(shape, Pn)
    o.init(phi, mu)
    o.step_phi_only()
    p, _ = o.download()
    assert np.abs(p.sum(0) - 1.0).max() < 1e-14


# --------------------------------------------------------------------------
# P3 + C.8: bulk exactness -- pure cells far from interfaces stay bitwise
# pure; a quiescent uniform solid keeps mu bitwise.
# --------------------------------------------------------------------------
def test_p3_bulk_exact(oracle_mod):
    shape = (24, 24, 24)
    phi, mu = I.ic_voronoi(shape, seed=3, nseeds=3, blur=1)
    o = oracle_mod.Oracle(shape, I.params_c4())
    o.init(phi, mu)
    nsteps = 3
    o.step(nsteps)
    p, _ = o.download()
    pure0 = phi.max(0) == 1.0
    far = pure0.copy()
    for ax in (0, 1, 2):  # cells whose (nsteps+1)-neighbourhood is pure at t = 0
        for s in range(1, nsteps + 2):
            far &= np.roll(pure0, s, ax) & np.roll(pure0, -s, ax)
    assert far.sum() > 100
    assert np.array_equal(p[:, far], phi[:, far])


def test_c8_quiescent_solid(oracle_mod):
    shape = (6, 6, 6)
    P = I.params_stress(G=0.0)
    phi = np.zeros((4,) + shape)
    phi[1] = 1.0
    mu = np.empty((2,) + shape)
    mu[0], mu[1] = 0.013, -0.007
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    o.step(3)
    p, m = o.download()
    assert np.array_equal(p, phi) and np.array_equal(m, mu)


# --------------------------------------------------------------------------
# P4: the 1-D two-phase sine profile phi = 1/2 + 1/2 sin(4x/(pi eps)) is the
# stationary solution of eqs. 4, 5, 7: the discrete
# residual inside the interface converges to 0 at second order.  A wrong
# coefficient anywhere in a2/a3 or omega' leaves an O(1) residual.
# --------------------------------------------------------------------------
def test_p4_sine_profile_stationary(oracle_mod):
    eps, L = 3.0, 40.0
    res = []
    for dx in [0.5, 0.25, 0.125]:
        nx = int(L / dx)
        x0 = L / 2 + 0.3 * dx
        u = (np.arange(nx) + 0.5) * dx - x0
        p1 = sine_profile(u, eps)
        phi = np.zeros((2, 1, 1, nx))
        phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
        dt = 0.05 * dx * dx
        o = oracle_mod.Oracle((1, 1, nx), simple_params(dx=dx, dt=dt), BC_X_NEUMANN)
        o.init(phi, np.zeros((1, 1, 1, nx)))
        o.step(1)
        p2, _ = o.download()
        r = np.abs(p2 - phi)[1, 0, 0] / dt
        inner = np.abs(u) < np.pi ** 2 * eps / 8 - 2 * dx
        res.append(r[inner].max())
    orders = np.log2(np.array(res[:-1]) / np.array(res[1:]))
    assert res[-1] < 5e-5
    assert np.all(orders > 1.8), (res, orders)


# --------------------------------------------------------------------------
# P5: third-phase suppression threshold gamma_abd > 32 gamma / pi^2 ~ 3.24
# (eq. 5 "higher order term to suppress spurious third-phases", P:L412-415;
# SURVEY App. A.2), with the Lagrange multiplier over all N phases [A3].
# --------------------------------------------------------------------------
@pytest.mark.parametrize("N", [3, 4])
def test_p5_third_phase_bound(oracle_mod, N):
    eps, dx, L = 3.0, 0.25, 30.0
    nx = int(L / dx)
    u = (np.arange(nx) + 0.5) * dx - (L / 2 + 0.3 * dx)
    p1 = sine_profile(u, eps)
    phi = np.zeros((N, 1, 1, nx))
    phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
    out = {}
    for g3 in (3.0, 3.5):
        o = oracle_mod.Oracle((1, 1, nx), simple_params(N=N, dx=dx, dt=0.05 * dx * dx, g3=g3), BC_X_NEUMANN)
        o.init(phi, np.zeros((1, 1, 1, nx)))
        o.step(20)
        p, _ = o.download()
        out[g3] = p[2:].max()
    assert out[3.0] > 1e-5      # below the bound a third phase appears
    assert out[3.5] == 0.0      # above it the projection keeps it exactly 0


# --------------------------------------------------------------------------
# P6: planar front speed v = d_psi / tau (from eqs. 6-7).
# --------------------------------------------------------------------------
def test_p6_front_velocity(oracle_mod):
    eps, dx, dpsi, tau, L = 3.0, 0.5, 0.03, 1.5, 40.0
    nx = int(L / dx)
    dt = 0.04 * dx * dx * tau
    u = (np.arange(nx) + 0.5) * dx - 12.0
    p1 = sine_profile(u, eps)
    phi = np.zeros((2, 1, 1, nx))
    phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
    o = oracle_mod.Oracle((1, 1, nx), simple_params(dx=dx, dt=dt, dpsi=dpsi, tau=tau), BC_X_NEUMANN)
    o.init(phi, np.zeros((1, 1, 1, nx)))
    o.step(int(30 / dt))
    f1 = front_position(o.download()[0][1, 0, 0], dx)
    n = int(60 / dt)
    o.step(n)
    f2 = front_position(o.download()[0][1, 0, 0], dx)
    v = (f2 - f1) / (n * dt)
    assert v / (dpsi / tau) == pytest.approx(1.0, abs=0.02)


# --------------------------------------------------------------------------
# A5: tau interpolation "computed from local phase-field values and pairwise
# kinetic coefficients tau_ab".  Whatever the interpolation, a
# binary a|b interface must move with its own pair's coefficient: the
# planar-front speed of App. A.3 is v = d_psi / tau_ab, independent of the
# tau of pairs that are absent.  Three phases with tau_01 = 2 and
# tau_02 = tau_12 = 1: the weighted mean gives tau = tau_01 exactly in every
# cell of the 0|1 front; an unweighted mean over all pairs would give 4/3
# (50 % faster); a max/min over all pairs 2 or 1.
# --------------------------------------------------------------------------
def test_a5_tau_binary_front_speed(oracle_mod):
    eps, dx, dpsi, L = 3.0, 0.5, 0.03, 40.0
    nx = int(L / dx)
    tau01 = 2.0
    dt = 0.04 * dx * dx
    u = (np.arange(nx) + 0.5) * dx - 12.0
    p1 = sine_profile(u, eps)
    phi = np.zeros((3, 1, 1, nx))
    phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
    P = simple_params(N=3, dx=dx, dt=dt, dpsi=dpsi, tau=1.0)
    P["tau"][0, 1] = P["tau"][1, 0] = tau01
    o = oracle_mod.Oracle((1, 1, nx), P, BC_X_NEUMANN)
    o.init(phi, np.zeros((1, 1, 1, nx)))
    o.step(int(30 / dt))
    f1 = front_position(o.download()[0][1, 0, 0], dx)
    n = int(60 / dt)
    o.step(n)
    p, _ = o.download()
    f2 = front_position(p[1, 0, 0], dx)
    assert p[2].max() == 0.0  # the third phase never appears (gamma3 = 10 > 32/pi^2)
    v = (f2 - f1) / (n * dt)
    assert v / (dpsi / tau01) == pytest.approx(1.0, abs=0.02)


def test_a5_tau_limits_in_cells(oracle_mod):
    """Delta-t linearity (C.8) isolates 1/tau per cell: without projection the
    phi increment is dt/(tau(phi) eps) R(phi), with R independent of tau.
    Against the same step with every tau_ab = 1 (tau = 1 exactly):
      - a cell where exactly two phases a, b are non-zero has tau = tau_ab
        (the binary-interface limit; to rounding);
      - every other mixed cell has tau inside [min, max] of the tau_ab of its
        present pairs (an interpolation of pairwise coefficients);
      - a pure cell (no pair present; reading A5's 0/0 case) uses the mean of
        all tau_ab."""
    shape = (10, 10, 10)
    P = I.params_stress()
    phi, mu = I.ic_voronoi(shape, seed=11, nseeds=12, blur=1, noise=0.0)
    outs = {}
    for name, tau in (("one", np.ones((4, 4)) - np.eye(4)), ("S", P["tau"])):
        o = oracle_mod.Oracle(shape, dict(P, tau=tau, projection=0))
        o.init(phi, mu)
        o.step_phi_only()
        outs[name] = o.download()[0] - phi
    T = P["tau"]
    present = phi > 0.0
    npres = present.sum(0)
    ok2 = okm = okp = 0
    for z, y, x in np.ndindex(*shape):
        a_ref, a_s = outs["one"][:, z, y, x], outs["S"][:, z, y, x]
        k = int(np.argmax(np.abs(a_ref)))
        if abs(a_ref[k]) < 1e-9:
            continue
        tau = a_ref[k] / a_s[k]  # tau(phi) / 1
        assert np.allclose(a_s * tau, a_ref, rtol=1e-12, atol=1e-15)  # one scalar per cell
        pr = np.nonzero(present[:, z, y, x])[0]
        pairs = [T[a, b] for i, a in enumerate(pr) for b in pr[i + 1:]]
        if npres[z, y, x] == 2:
            assert tau == pytest.approx(pairs[0], rel=1e-12)
            ok2 += 1
        elif npres[z, y, x] > 2:
            assert min(pairs) * (1 - 1e-12) <= tau <= max(pairs) * (1 + 1e-12)
            okm += 1
        else:
            assert tau == pytest.approx(T[np.triu_indices(4, 1)].mean(), rel=1e-12)
            okp += 1
    assert ok2 > 20 and okm > 20 and okp > 20, (ok2, okm, okp)


# --------------------------------------------------------------------------
# A15: Dirichlet mu = mu_inf at z_hi (DS boundaries), Neumann at z_lo.  Pure
# liquid, uniform mu0 != mu_inf, dT/dt = 0: the mu equation is FTCS diffusion
# (App. A.4) whose only source is the top face, between the top cell and a
# ghost holding mu_inf (C.6.6).  One step changes only the top cell:
#   mu'_top = mu0 + (dt/dx^2) K (mu_inf - mu0),  K = chi_l^{-1} D_l chi_l,
# and a second step reaches the cell below by the same factor.
# --------------------------------------------------------------------------
def test_a15_dirichlet_mu_top(oracle_mod):
    P = I.params_stress(G=0.0, v=0.0)
    P["mu_inf"] = np.array([0.03, -0.02])
    shape = (6, 3, 4)
    mu0 = np.array([0.01, 0.005])
    phi = np.zeros((4,) + shape)
    phi[3] = 1.0
    mu = np.zeros((2,) + shape) + mu0[:, None, None, None]
    o = oracle_mod.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    o.step(1)
    p, m = o.download()
    A = P["A0"][3] + P["A1"][3] * P["T0"]
    chi = -(A + A.T)
    K = np.linalg.solve(chi, P["D"][3] @ chi) * P["dt"] / P["dx"] ** 2
    top = mu0 + K @ (P["mu_inf"] - mu0)
    assert np.array_equal(p, phi)
    assert np.array_equal(m[:, :-1], mu[:, :-1])  # Neumann bottom, untouched interior
    for i in range(2):
        np.testing.assert_allclose(m[i, -1], top[i], rtol=0, atol=1e-16)
    o.step(1)
    _, m2 = o.download()
    below = mu0 + K @ (top - mu0)
    top2 = top + K @ (P["mu_inf"] - top) - K @ (top - mu0)
    for i in range(2):
        np.testing.assert_allclose(m2[i, -2], below[i], rtol=0, atol=1e-16)
        np.testing.assert_allclose(m2[i, -1], top2[i], rtol=0, atol=1e-16)
    assert np.array_equal(m2[:, :-2], mu[:, :-2])


# --------------------------------------------------------------------------
# P7: r_a = delta Psi / delta phi_a of the oracle converges at second order
# to sympy's variational derivative of eq. 3 (the paper's own route,
# `func_diff`), on smooth periodic fields.
# --------------------------------------------------------------------------
def _sympy_rhs(P, Lbox):
    import sympy as sp
    N, M = P["N"], P["M"]
    X = sp.symbols("x y z", real=True)
    u = sp.symbols(f"u0:{N}", real=True)
    g = [[sp.Symbol(f"p{a}_{d}", real=True) for d in range(3)] for a in range(N)]
    m = sp.symbols(f"m0:{M}", real=True)
    eps = sp.Float(P["eps"])
    # eq. 4 with A_ab = 1 (P1), q_ab = u_a grad u_b - u_b grad u_a [A2]
    a_ = 0
    for al in range(N):
        for be in range(al + 1, N):
            q = [u[al] * g[be][d] - u[be] * g[al][d] for d in range(3)]
            a_ += sp.Float(P["gamma"][al, be]) * sum(c * c for c in q)
    # eq. 5
    om = 0
    for al in range(N):
        for be in range(al + 1, N):
            om += 16 / sp.pi ** 2 * sp.Float(P["gamma"][al, be]) * u[al] * u[be]
            for de in range(be + 1, N):
                om += sp.Float(P["gamma3"][al, be, de]) * u[al] * u[be] * u[de]
    # eq. 6 with h(u) = u^2 (3 - 2u) [A4], constant T
    T = P["T0"]
    psi = 0
    for al in range(N):
        A = P["A0"][al] + P["A1"][al] * T
        B = P["B0"][al] + P["B1"][al] * T
        Cc = P["C0"][al] + P["C1"][al] * T
        pa = sum(m[i] * sp.Float(A[i, j]) * m[j] for i in range(M) for j in range(M))
        pa += sum(sp.Float(B[i]) * m[i] for i in range(M)) + sp.Float(Cc)
        psi += pa * u[al] ** 2 * (3 - 2 * u[al])
    f = eps * a_ + om / eps + psi
    # smooth periodic fields (not on the simplex: r_a does not need it)
    k = 2 * sp.pi / Lbox
    phis = [sp.Rational(1, 4) + sp.Rational(1, 5) * sp.sin(k * X[0] + a) * sp.cos(k * X[1] + 2 * a)
            + sp.Rational(1, 10) * sp.cos(k * X[2] + 0.5 * a) for a in range(N)]
    mus = [sp.Rational(1, 20) * sp.sin(k * (X[0] + X[1]) + i) * sp.cos(k * X[2]) for i in range(M)]
    sub = {u[a]: phis[a] for a in range(N)}
    sub.update({g[a][d]: sp.diff(phis[a], X[d]) for a in range(N) for d in range(3)})
    sub.update({m[i]: mus[i] for i in range(M)})
    rhs = []
    for al in range(N):
        e = sp.diff(f, u[al]).subs(sub)
        for d in range(3):
            e -= sp.diff(sp.diff(f, g[al][d]).subs(sub), X[d])
        rhs.append(sp.lambdify(X, e, "numpy"))
    fphi = [sp.lambdify(X, p, "numpy") for p in phis]
    fmu = [sp.lambdify(X, q, "numpy") for q in mus]
    return rhs, fphi, fmu


def test_p7_sympy_variational_derivative(oracle_mod):
    P = I.params_stress(G=0.0)
    Lbox = 16.0
    rhs, fphi, fmu = _sympy_rhs(P, Lbox)
    errs = []
    for n in (8, 16, 32):
        dx = Lbox / n
        c = (np.arange(n) + 0.5) * dx
        Z, Y, X = np.meshgrid(c, c, c, indexing="ij")
        phi = np.stack([np.broadcast_to(f(X, Y, Z), X.shape) for f in fphi]).astype(np.float64)
        mu = np.stack([np.broadcast_to(f(X, Y, Z), X.shape) for f in fmu]).astype(np.float64)
        o = oracle_mod.Oracle((n, n, n), dict(P, dx=dx))
        o.init(phi, mu)
        r = o.phi_rhs()
        ref = np.stack([np.broadcast_to(f(X, Y, Z), X.shape) for f in rhs])
        errs.append(np.abs(r - ref).max() / np.abs(ref).max())
    orders = np.log2(np.array(errs[:-1]) / np.array(errs[1:]))
    assert errs[-1] < 2e-3 and np.all(np.abs(orders - 2.0) < 0.2), (errs, orders)


# --------------------------------------------------------------------------
# P8: uniform pure liquid, sinusoidal mu: the mu step is FTCS diffusion with
# D_l (eqs. 8-9): exact per-step amplitude factor
# lambda = 1 - (4 D dt / dx^2) sum_d sin^2(pi m_d / n_d).
# --------------------------------------------------------------------------
def test_p8_mu_fourier_decay(oracle_mod):
    P = I.params_stress(G=0.0)
    Dl = 0.37
    P["D"][3] = Dl * np.eye(2)
    P["dt"] = 0.05
    shape = (16, 8, 12)  # nz, ny, nx
    mvec = (1, 2, 3)     # (mz, my, mx)
    z, y, x = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
    wave = np.cos(2 * np.pi * (mvec[0] * z / shape[0] + mvec[1] * y / shape[1] + mvec[2] * x / shape[2]) + 0.3)
    mu0 = np.array([0.02, -0.01])
    mu = np.stack([mu0[0] + 0.01 * wave, mu0[1] - 0.004 * wave])
    phi = np.zeros((4,) + shape)
    phi[3] = 1.0
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    o.step(1)
    p, m = o.download()
    lam = 1.0 - 4.0 * Dl * P["dt"] / P["dx"] ** 2 * sum(
        np.sin(np.pi * md / nd) ** 2 for md, nd in zip(mvec, shape))
    assert np.array_equal(p, phi)
    for i in range(2):
        np.testing.assert_allclose(m[i] - mu0[i], lam * (mu[i] - mu0[i]), rtol=0, atol=1e-15)


def test_p8_product_order_D_chi(oracle_mod):
    """P8 with non-commuting D_l and chi_l [A7]: the Fourier mode evolves by
    the exact matrix factor I - (4 dt/dx^2) sum sin^2 * chi^{-1} D chi."""
    P = I.params_stress(G=0.0)
    P["dt"] = 0.05
    D = np.array([[0.5, 0.2], [-0.1, 0.3]])
    P["D"][3] = D
    shape = (8, 6, 10)
    mvec = (1, 1, 2)
    z, y, x = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
    wave = np.sin(2 * np.pi * sum(m * c / n for m, c, n in zip(mvec, (z, y, x), shape)) + 0.7)
    amp = np.array([0.01, 0.006])
    mu = amp[:, None, None, None] * wave
    phi = np.zeros((4,) + shape)
    phi[3] = 1.0
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    o.step(1)
    _, m = o.download()
    A = P["A0"][3] + P["A1"][3] * P["T0"]
    chi = -(A + A.T)
    s = 4.0 * P["dt"] / P["dx"] ** 2 * sum(np.sin(np.pi * md / nd) ** 2 for md, nd in zip(mvec, shape))
    Fm = np.eye(2) - s * np.linalg.solve(chi, D @ chi)
    expect = np.einsum("ij,j...->i...", Fm, mu)
    np.testing.assert_allclose(m, expect, rtol=0, atol=1e-15)


def test_mobility_face_interpolation(oracle_mod):
    """eq. 9 with g_a = phi_a [A4] at the face mean [A9]: across a static 1-D
    interface (equal psi_a, so phi and c do not move) a linear mu is plain
    variable-coefficient diffusion; the telescoped face flux divided by the
    gradient is the face mobility M = sum_a D_a chi_a g(phibar_a)."""
    eps, dx, nx = 3.0, 0.5, 60
    u = (np.arange(nx) + 0.5) * dx - nx * dx / 2
    p1 = sine_profile(u, eps)
    phi = np.zeros((2, 1, 1, nx))
    phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
    P = simple_params(dx=dx, dt=0.01)
    Ds, Dl, a = 0.1, 1.0, 0.02
    P["D"] = np.array([[[Ds]], [[Dl]]])
    mu = (a * (np.arange(nx) + 0.5) * dx)[None, None, None, :].copy()
    o = oracle_mod.Oracle((1, 1, nx), P, BC_X_NEUMANN)
    o.init(phi, mu)
    o.step(1)
    p2, m2 = o.download()
    assert np.abs(p2 - phi).max() < 1e-3
    F = (dx / P["dt"]) * np.cumsum((m2 - mu)[0, 0, 0])[:-1]  # chi = h(phi)+h(1-phi) = 1
    pb = 0.5 * (phi[:, 0, 0, :-1] + phi[:, 0, 0, 1:])
    Mf = Ds * pb[0] + Dl * pb[1]
    np.testing.assert_allclose(F / a, Mf, rtol=1e-10, atol=1e-12)


def test_mobility_temperature_at_faces(oracle_mod):
    """Frozen T (A13) evaluated on staggered z-faces at z = k + 1/2: in pure
    liquid with A1 != 0 and v = 0, a mu linear in z diffuses with the face
    mobility D chi_l(T(k+1/2)); chi at the cell uses T(k)."""
    P = I.params_stress(v=0.0)
    P["D"][3] = 0.4 * np.eye(2)
    L, nz = 3, 12
    shape = (nz, 3, 4)
    bc = {"lo": ("periodic", "periodic", "neumann"), "hi": ("periodic", "periodic", "neumann")}
    grad = np.array([0.01, -0.004])
    k = np.arange(nz)
    mu = np.zeros((2,) + shape) + (grad[:, None] * (k + 0.5))[:, :, None, None]
    phi = np.zeros((4,) + shape)
    phi[3] = 1.0
    o = oracle_mod.Oracle(shape, P, bc)
    o.init(phi, mu)
    o.step(1)
    _, m = o.download()
    T = lambda zz: P["T0"] + P["G"] * zz * P["dx"]
    chi = lambda t: -((P["A0"][L] + P["A1"][L] * t) + (P["A0"][L] + P["A1"][L] * t).T)
    # telescope chi(T_k)(mu' - mu) dx / dt from the bottom (Neumann: zero flux)
    acc = np.zeros(2)
    for kk in range(nz - 1):
        acc = acc + chi(T(kk)) @ (m[:, kk, 0, 0] - mu[:, kk, 0, 0]) * P["dx"] / P["dt"]
        expect = 0.4 * chi(T(kk + 0.5)) @ grad / P["dx"]
        np.testing.assert_allclose(acc, expect, rtol=1e-10, atol=1e-15)


# --------------------------------------------------------------------------
# P9: frozen temperature (A13) and the Q-term of eq. 8: a uniform pure-liquid
# state with G v != 0 follows the single-cell ODE
#   mu' - mu = -dt chi_l(T_k)^{-1} (dc_l/dT) dT/dt,  dT/dt = -G v.
# --------------------------------------------------------------------------
def test_p9_temperature_Q_term(oracle_mod):
    P = I.params_stress()
    shape = (10, 3, 4)
    mu0 = np.array([0.03, -0.02])
    phi = np.zeros((4,) + shape)
    phi[3] = 1.0
    mu = np.empty((2,) + shape)
    mu[0], mu[1] = mu0
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    o.set_state(step=7, z_off=5)
    o.step(1)
    _, m = o.download()
    L = 3
    dTdt = -P["G"] * P["v"]
    for k in range(shape[0]):
        T = P["T0"] + P["G"] * ((k + 5) * P["dx"] - P["v"] * 7 * P["dt"])
        A = P["A0"][L] + P["A1"][L] * T
        chi = -(A + A.T)
        dcdT = -(P["A1"][L] + P["A1"][L].T) @ mu0 - P["B1"][L]
        expect = mu0 - P["dt"] * np.linalg.solve(chi, dcdT * dTdt)
        for i in range(2):
            assert np.abs(m[i, k] - expect[i]).max() < 1e-16 + 1e-14 * abs(expect[i])


# --------------------------------------------------------------------------
# P10: exact discrete solute identity under periodic BCs with dT/dt = 0:
#   sum_cells [ chi (mu' - mu) + sum_a c_a h'_a (phi'_a - phi_a) ] = 0
# -- the mu fluxes (M grad mu - J_at, eqs. 8-10) telescope.
# --------------------------------------------------------------------------
@pytest.mark.parametrize("ic", ["R", "V"])
def test_p10_solute_flux_identity(oracle_mod, ic):
    P = I.params_stress(G=0.0, v=0.0)  # T must be periodic for the fluxes to telescope
    shape = (8, 9, 10)
    phi, mu = I.make_ic(ic, shape, seed=5)
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    o.step(1)
    p2, m2 = o.download()
    N, M = 4, 2
    k = np.arange(shape[0])[:, None, None]
    T = P["T0"] + P["G"] * k * P["dx"] + 0 * phi[0]
    tot = np.zeros(M)
    scale = np.zeros(M)
    for a in range(N):
        A = P["A0"][a][:, :, None, None, None] + P["A1"][a][:, :, None, None, None] * T
        B = P["B0"][a][:, None, None, None] + P["B1"][a][:, None, None, None] * T
        chi = -(A + A.transpose(1, 0, 2, 3, 4))  # c = -(A + A^T) mu - B   [A6]
        c = -np.einsum("ij...,j...->i...", A + A.transpose(1, 0, 2, 3, 4), mu) - B
        h = phi[a] ** 2 * (3 - 2 * phi[a])
        dh = 6 * phi[a] * (1 - phi[a])
        t1 = np.einsum("ij...,j...->i...", h * chi, m2 - mu)
        t2 = c * dh * (p2[a] - phi[a])
        tot += (t1 + t2).sum(axis=(1, 2, 3))
        scale += (np.abs(t1) + np.abs(t2)).sum(axis=(1, 2, 3))
    assert np.all(np.abs(tot) <= 1e-13 * scale), (tot, scale)


# --------------------------------------------------------------------------
# Anti-trapping current J_at (eq. 10) against its travelling-wave
# closed form.  On the stationary profile (pi eps/4)|grad phi|/sqrt(phi(1-phi)) = 1,
# and d_t phi = v |grad phi| for a front moving at v, so eq. 10 reduces to
#   J_at = v (c_l - c_a) phi_a h(phi_l) n     (n = growth direction).
# The oracle's J is read back from mu (antitrapping on minus off) by summing
# the telescoping divergence.  1-D front: prefactor, weight, dot product and
# sign; diagonal front: the tangential face derivatives (eq. 11, A9) in n.
# --------------------------------------------------------------------------
def _front_run(oracle_mod, shape, P, phi, bc, steps_warm, steps_meas, front_of):
    o = oracle_mod.Oracle(shape, P, bc)
    o.init(phi, np.zeros((1,) + shape))
    o.step(steps_warm)
    f1 = front_of(o.download()[0])
    o.step(steps_meas)
    p, m = o.download()
    f2 = front_of(p)
    return p, m, (f2 - f1) / (steps_meas * P["dt"])


def _J_from_mu(oracle_mod, shape, P, p, m, bc, dc):
    out = {}
    for at in (0, 1):
        Q = dict(P, antitrapping=at, B0=np.array([[0.0], [-dc]]))
        q = oracle_mod.Oracle(shape, Q, bc)
        q.init(p, m)
        q.step(1)
        out[at] = q.download()[1][0]
    return out[1] - out[0]


def test_antitrapping_1d_closed_form(oracle_mod):
    eps, dx, dpsi, L, dc = 3.0, 0.5, 0.03, 40.0, 0.5
    nx = int(L / dx)
    dt = 0.04 * dx * dx
    u = (np.arange(nx) + 0.5) * dx - 12.0
    p1 = sine_profile(u, eps)
    phi = np.zeros((2, 1, 1, nx))
    phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
    P = simple_params(dx=dx, dt=dt, dpsi=dpsi)
    p, m, v = _front_run(oracle_mod, (1, 1, nx), P, phi, BC_X_NEUMANN, int(40 / dt), int(20 / dt),
                         lambda q: front_position(q[1, 0, 0], dx))
    assert np.all(m == 0.0)
    d = _J_from_mu(oracle_mod, (1, 1, nx), P, p, m, BC_X_NEUMANN, dc)[0, 0]
    J = -(dx / dt) * np.cumsum(d)[:-1]                 # J at faces i+1/2 (chi = 1)
    ps = 0.5 * (p[0, 0, 0, :-1] + p[0, 0, 0, 1:])
    pl = 1.0 - ps
    Jc = v * dc * ps * pl * pl * (3 - 2 * pl)
    assert np.abs(J - Jc).max() < 0.05 * Jc.max()


def test_antitrapping_diagonal_front(oracle_mod):
    eps, dx, dpsi, dc = 3.0, 1.0, 0.03, 0.5
    n = 48
    dt = 0.04
    i = np.arange(n)
    s = ((i[None, :] + i[:, None]) % n) * dx          # [y][x], s = x + y
    dist = (s - n * dx / 2) / np.sqrt(2)                # signed distance along n = (1,1)/sqrt2
    ps = sine_profile(6.0 - np.abs(dist), eps)          # solid slab, two fronts
    phi = np.zeros((2, 1, n, n))
    phi[0, 0], phi[1, 0] = ps, 1.0 - ps
    P = simple_params(dx=dx, dt=dt, dpsi=dpsi)
    p, m, vs = _front_run(oracle_mod, (1, n, n), P, phi, BC_PERIODIC, int(10 / dt), int(5 / dt),
                          lambda q: front_position(q[1, 0, 0], dx, start=n // 2))
    v = vs / np.sqrt(2)                                  # normal speed from the speed along x
    d = _J_from_mu(oracle_mod, (1, n, n), P, p, m, BC_PERIODIC, dc)[0, 0, n // 2:]
    J = -(dx / (2 * dt)) * np.cumsum(d)[:-1]           # div = 2 dJ/ds along the x axis
    sol = 0.5 * (p[0, 0, 0, n // 2:-1] + p[0, 0, 0, n // 2 + 1:])
    pl = 1.0 - sol
    Jc = v * dc * sol * pl * pl * (3 - 2 * pl) / np.sqrt(2)   # x-component
    assert np.abs(J - Jc).max() < 0.08 * Jc.max()


# --------------------------------------------------------------------------
# P12: symmetries.
# --------------------------------------------------------------------------
def _run(oracle_mod, P, phi, mu, steps=2, bc=None):
    o = oracle_mod.Oracle(phi.shape[1:], P, bc)
    o.init(phi, mu)
    o.step(steps)
    return o.download()


def test_p12_translation_bitwise(oracle_mod):
    P = I.params_stress(G=0.0, v=0.0)
    phi, mu = I.ic_voronoi((8, 10, 12), seed=7)
    p1, m1 = _run(oracle_mod, P, phi, mu)
    sh = (3, 2, 1)
    roll = lambda a: np.roll(a, sh, axis=(1, 2, 3))
    p2, m2 = _run(oracle_mod, P, roll(phi), roll(mu))
    assert np.array_equal(roll(p1), p2) and np.array_equal(roll(m1), m2)


def test_p12_mirror_and_axis_permutation(oracle_mod):
    P = I.params_stress()  # G != 0: z is special, x and y are not
    phi, mu = I.ic_voronoi((8, 10, 10), seed=8)
    p1, m1 = _run(oracle_mod, P, phi, mu)
    fx = lambda a: a[..., ::-1].copy()
    p2, m2 = _run(oracle_mod, P, fx(phi), fx(mu))
    np.testing.assert_allclose(fx(p1), p2, atol=1e-14, rtol=0)
    np.testing.assert_allclose(fx(m1), m2, atol=1e-14, rtol=0)
    tr = lambda a: a.transpose(0, 1, 3, 2).copy()
    p3, m3 = _run(oracle_mod, P, tr(phi), tr(mu))
    np.testing.assert_allclose(tr(p1), p3, atol=1e-14, rtol=0)
    np.testing.assert_allclose(tr(m1), m3, atol=1e-14, rtol=0)


def test_p12_solid_phase_permutation(oracle_mod):
    P = I.params_stress()
    phi, mu = I.ic_voronoi((8, 8, 8), seed=9)
    perm = np.array([2, 0, 1, 3])  # new phase k = old phase perm[k]; liquid fixed
    Q = dict(P)
    for key in ("A0", "A1", "B0", "B1", "C0", "C1", "D"):
        Q[key] = P[key][perm]
    Q["gamma"] = P["gamma"][np.ix_(perm, perm)]
    Q["tau"] = P["tau"][np.ix_(perm, perm)]
    Q["gamma3"] = P["gamma3"][np.ix_(perm, perm, perm)]
    p1, m1 = _run(oracle_mod, P, phi, mu)
    p2, m2 = _run(oracle_mod, Q, phi[perm], mu)
    np.testing.assert_allclose(p1[perm], p2, atol=1e-14, rtol=0)
    np.testing.assert_allclose(m1, m2, atol=1e-14, rtol=0)


# --------------------------------------------------------------------------
# P15: gradient-flow sign (eq. 7 + listing, [A1]): with mu frozen the
# discrete energy of eq. 3 decreases monotonically.
# --------------------------------------------------------------------------
def _energy(phi, mu, P):
    N, M, dx, eps = P["N"], P["M"], P["dx"], P["eps"]
    g = [[(np.roll(phi[a], -1, ax) - np.roll(phi[a], 1, ax)) / (2 * dx) for ax in (0, 1, 2)] for a in range(N)]
    e = 0.0
    for al in range(N):
        for be in range(al + 1, N):
            q2 = sum((phi[al] * g[be][d] - phi[be] * g[al][d]) ** 2 for d in range(3))
            e = e + eps * P["gamma"][al, be] * q2 + 16 / np.pi ** 2 / eps * P["gamma"][al, be] * phi[al] * phi[be]
            for de in range(be + 1, N):
                e = e + P["gamma3"][al, be, de] * phi[al] * phi[be] * phi[de] / eps
    T = P["T0"]
    for al in range(N):
        A, B = P["A0"][al] + P["A1"][al] * T, P["B0"][al] + P["B1"][al] * T
        ps = sum(mu[i] * A[i, j] * mu[j] for i in range(M) for j in range(M)) + sum(B[i] * mu[i] for i in range(M))
        ps = ps + P["C0"][al] + P["C1"][al] * T
        e = e + ps * phi[al] ** 2 * (3 - 2 * phi[al])
    return float(np.sum(e))


@pytest.mark.parametrize("ic", ["R", "V"])
def test_p15_energy_decay(oracle_mod, ic):
    P = I.params_c4()
    phi, mu = I.make_ic(ic, (12, 12, 12), seed=1)
    o = oracle_mod.Oracle((12, 12, 12), P)
    o.init(phi, mu)
    E = [_energy(phi, mu, P)]
    for _ in range(15):
        o.step_phi_only()
        p, m = o.download()
        assert np.array_equal(m, mu)
        E.append(_energy(p, m, P))
    assert np.all(np.diff(E) < 0), E


# --------------------------------------------------------------------------
# Host logic of the oracle: OpenMP bitwise == serial; moving window (A16).
# --------------------------------------------------------------------------
def test_openmp_bitwise(oracle_mod):
    P = I.params_stress()
    phi, mu = I.ic_random((6, 7, 8), seed=4)
    ref = _run(oracle_mod, P, phi, mu, steps=2)
    oracle_mod.set_threads(4)
    try:
        got = _run(oracle_mod, P, phi, mu, steps=2)
    finally:
        oracle_mod.set_threads(0)
    assert np.array_equal(ref[0], got[0]) and np.array_equal(ref[1], got[1])


def test_window_shift_semantics(oracle_mod):
    P = I.params_c4("ds", window_check=0, mu_inf=np.array([0.02, -0.01]))
    shape = (16, 6, 8)
    phi, mu = I.ic_lamellar(shape, seed=3, z_front=10, mu_inf=(0.005, 0.004))
    o = oracle_mod.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    H = o.front_height()
    assert H == np.nonzero((phi[3] < 0.5).any(axis=(1, 2)))[0].max()
    o.shift_window(3)
    p, m = o.download()
    assert np.array_equal(p[:, :-3], phi[:, 3:]) and np.array_equal(m[:, :-3], mu[:, 3:])
    assert np.all(p[3, -3:] == 1.0) and np.all(p[:3, -3:] == 0.0)
    assert np.all(m[0, -3:] == 0.02) and np.all(m[1, -3:] == -0.01)  # inflow mu = mu_inf [A16]
    assert o.state()["z_off"] == 3


def test_window_auto_trigger(oracle_mod):
    P = I.params_c4("ds", window_check=2, window_frac=0.5)
    shape = (16, 6, 8)
    phi, mu = I.ic_lamellar(shape, seed=3, z_front=12)
    o = oracle_mod.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    o.step(2)
    st = o.state()
    assert st["z_off"] > 0 and o.front_height() <= 8


# --------------------------------------------------------------------------
# Fluctuation term xi (eq. 7 "+ xi(phi)", listing P:L490-495:
# fluctuation = amplitude * random(-1, 1, kind='philox'); RNG P:L669-676),
# reading B4: xi_a = A U_a, U_a = (u_a + 1/2) 2^-31 - 1 from Philox4x32-10
# with counter (x, y, z, step) and key (seed, step >> 32).
# --------------------------------------------------------------------------
def _kat():
    rows = []
    for ln in open(os.path.join(GOLDEN, "philox4x32_10_kat.txt")):
        if ln.strip() and not ln.startswith("#"):
            w = [int(t, 16) for t in ln.split()]
            rows.append((w[0:4], w[4:6], tuple(w[6:10])))
    return rows


def test_xi_philox_known_answers(oracle_mod):
    """The oracle's Philox4x32-10 reproduces the published known-answer vectors."""
    for ctr, key, out in _kat():
        assert oracle_mod.philox4x32_10(ctr, key) == out


def test_xi_uniforms_distribution(oracle_mod):
    """U in (-1, 1): mean 0, variance 1/3, the four phases uncorrelated, a new
    draw every step (counter = cell and step)."""
    rng = np.random.default_rng(5)
    cells = rng.integers(0, 400, size=(4000, 3))
    U = np.array([oracle_mod.xi_uniforms(x, y, z, 7, 20191117) for x, y, z in cells])
    assert np.all(np.abs(U) < 1.0)
    assert np.abs(U.mean(0)).max() < 0.04
    assert np.abs(U.var(0) - 1.0 / 3.0).max() < 0.03
    C = np.corrcoef(U.T)
    assert np.abs(C - np.eye(4)).max() < 0.06
    V = np.array([oracle_mod.xi_uniforms(x, y, z, 8, 20191117) for x, y, z in cells])
    assert np.abs(np.corrcoef(U[:, 0], V[:, 0])[0, 1]) < 0.06
    # the mapping of the 32-bit words: u = 0 -> -1 + 2^-32, u = 2^32 - 1 -> 1 - 2^-32
    words = oracle_mod.philox4x32_10((3, 4, 5, 6), (99, 0))
    expect = np.array([(w + 0.5) / 2.0 ** 31 - 1.0 for w in words])
    assert np.array_equal(oracle_mod.xi_uniforms(3, 4, 5, 6, 99), expect)


def test_xi_enters_the_euler_step(oracle_mod):
    """With all tau_ab equal (tau = tau0 exactly) and no projection, one step
    with amplitude A differs from the step without noise by exactly
    dt/(tau0 eps) A U_a(x, y, z, n=0) per phase (the noise is added to the
    right-hand side of eq. 7, outside the Lagrange multiplier)."""
    shape = (5, 6, 7)
    P = I.params_stress()
    P["tau"] = np.full((4, 4), 1.7)
    phi, mu = I.ic_voronoi(shape, seed=9)
    outs = []
    for A in (0.0, 0.05):
        o = oracle_mod.Oracle(shape, dict(P, projection=0, xi_amp=A, xi_seed=77))
        o.init(phi, mu)
        o.step_phi_only()
        outs.append(o.download()[0])
    f = P["dt"] / (1.7 * P["eps"])
    z, y, x = np.meshgrid(range(shape[0]), range(shape[1]), range(shape[2]), indexing="ij")
    U = np.array([oracle_mod.xi_uniforms(a, b, c, 0, 77) for a, b, c in zip(x.ravel(), y.ravel(), z.ravel())])
    U = U.T.reshape((4,) + shape)
    assert np.abs((outs[1] - outs[0]) - f * 0.05 * U).max() < 1e-15


def test_xi_invariants_and_bulk(oracle_mod):
    """With noise: sum phi = 1 and phi >= 0 every step (P2); an amplitude
    below the obstacle margin keeps bulk cells bitwise pure (P3): in a pure
    cell the other phases receive dt/(tau eps) (mean r - r_b + xi_b) < 0
    when A < (16 gamma / pi^2)/(4 eps) (eq. 5)."""
    shape = (24, 24, 24)
    P = I.params_c4()
    phi, mu = I.ic_voronoi(shape, seed=3, nseeds=3, blur=1)
    A = 0.5 * (16.0 / np.pi ** 2) / (4.0 * P["eps"])
    o = oracle_mod.Oracle(shape, dict(P, xi_amp=A, xi_seed=5))
    o.init(phi, mu)
    for _ in range(3):
        o.step(1)
        p, _ = o.download()
        assert np.abs(p.sum(0) - 1.0).max() <= 8 * 2.2e-16
        assert p.min() >= 0.0
    pure0 = phi.max(0) == 1.0
    far = pure0.copy()
    for ax in (0, 1, 2):
        for s in range(1, 5):
            far &= np.roll(pure0, s, ax) & np.roll(pure0, -s, ax)
    assert far.sum() > 100
    assert np.array_equal(p[:, far], phi[:, far])
    # and the noise does act in the interfaces
    o2 = oracle_mod.Oracle(shape, P)
    o2.init(phi, mu)
    o2.step(3)
    assert np.abs(o2.download()[0] - p).max() > 1e-4
