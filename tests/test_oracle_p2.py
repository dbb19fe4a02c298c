"""Pins of the oracle's P2 parameterisation (SURVEY §8(f) NEXT-4,
P:L1199-1213): 3 phases, 2 components (one chemical potential), anisotropic
gradient energy a = sum_{a<b} gamma_ab A_ab(R_ab q_ab)^2 |q_ab|^2 (eq. 4,
P:L382-398) with the cubic A of reading B6.  CPU only (-m "not gpu").

What fixes the anisotropic part independently of the oracle's code:
  - Table 1's P2 load / store counts (the 19-point phi stencil);
  - the planar two-phase profile along a direction n is the P1 sine profile
    with the gradient coefficient gamma A(R n)^2, i.e. its width scales with
    A (App. A.1 with gamma_grad = gamma A^2);
  - sympy's derivatives of the anisotropic pair energy f(q) = A(Rq)^2 |q|^2
    composed into the continuum variational derivative (the paper's route,
    P:L490): second-order convergence of r_a;
  - rotating the lattice by 90 degrees together with R -> R Q^T commutes
    with the step; delta = 0 is the isotropic P1 step.
"""
import json
import os

import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I
from tests._pins_common import BC_X_NEUMANN, simple_params

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def cubic_A(delta, n):
    """A(n) = 1 - delta (3 - 4 sum_i n_i^4 / |n|^4) (reading B6), written out."""
    n = np.asarray(n, dtype=float)
    return 1.0 - delta * (3.0 - 4.0 * np.sum(n ** 4) / np.sum(n ** 2) ** 2)


def test_p2_table1_footprint(oracle_mod):
    gold = json.load(open(os.path.join(GOLDEN, "table1_p2.json")))
    P = I.params_p2()
    shape = (6, 6, 6)
    phi, mu = I.ic_random(shape, seed=3, N=3, M=1)
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    for k in gold["loads"]:
        loads, stores = o.footprint(k, (2, 3, 2))
        assert loads == gold["loads"][k], (k, loads)
        assert stores == gold["stores"][k], (k, stores)


def test_p2_delta0_is_isotropic(oracle_mod):
    P = I.params_p2_stress()
    shape = (8, 9, 10)
    phi, mu = I.ic_voronoi(shape, seed=4, N=3, M=1)
    outs = []
    for aniso in (0, 1):
        Q = dict(P, aniso=aniso, aniso_delta=np.zeros((3, 3)))
        o = oracle_mod.Oracle(shape, Q)
        o.init(phi, mu)
        o.step(2)
        outs.append(o.download())
    for a, b in zip(outs[0], outs[1]):
        assert np.abs(a - b).max() <= 1e-14 * np.abs(a).max()


@pytest.mark.parametrize("Rspec", [("z", 0.0), ("z", 45.0), ("y", -40.0)])
def test_p2_planar_profile_width(oracle_mod, Rspec):
    """Two phases, a planar profile along x: q = -grad phi is parallel to
    e_x, so the anisotropic functional is the isotropic one with gradient
    coefficient gamma A(R e_x)^2.  The stationary profile is the App. A.1
    sine with k = 4 / (pi eps A): its residual converges at second order,
    the unscaled profile's does not."""
    eps, L, delta = 3.0, 40.0, 0.06
    R = I.rot(*Rspec) @ I.rot("x", 15.0)
    Aex = cubic_A(delta, R @ np.array([1.0, 0.0, 0.0]))
    assert abs(Aex - 1.0) > 0.01
    res = {True: [], False: []}
    for dx in (0.5, 0.25, 0.125):
        nx = int(L / dx)
        u = (np.arange(nx) + 0.5) * dx - (L / 2 + 0.3 * dx)
        for scaled in (True, False):
            ee = eps * Aex if scaled else eps
            k = 4.0 / (np.pi * ee)
            w = np.pi / (2.0 * k)
            p1 = np.where(u < -w, 0.0, np.where(u > w, 1.0, 0.5 + 0.5 * np.sin(k * np.clip(u, -w, w))))
            phi = np.zeros((2, 1, 1, nx))
            phi[1, 0, 0], phi[0, 0, 0] = p1, 1.0 - p1
            dt = 0.05 * dx * dx
            P = simple_params(dx=dx, dt=dt)
            P.update(aniso=1, aniso_delta=np.array([[0.0, delta], [delta, 0.0]]),
                     aniso_R=np.array([[np.eye(3), R], [R, np.eye(3)]]))
            o = oracle_mod.Oracle((1, 1, nx), P, BC_X_NEUMANN)
            o.init(phi, np.zeros((1, 1, 1, nx)))
            o.step(1)
            p2, _ = o.download()
            r = np.abs(p2 - phi)[1, 0, 0] / dt
            inner = np.abs(u) < w - 2 * dx
            res[scaled].append(r[inner].max())
    orders = np.log2(np.array(res[True][:-1]) / np.array(res[True][1:]))
    assert res[True][-1] < 1e-4 and np.all(orders > 1.8), (res[True], orders)
    assert res[False][-1] > 20 * res[True][-1], (res[False], res[True])


def test_p2_lattice_rotation_covariance(oracle_mod):
    """Rotate the periodic box by 90 degrees about z (x' = n-1-y, y' = x)
    and every R_ab -> R_ab Q^T (Q the rotation of the coordinates): the step
    commutes with the rotation (to rounding)."""
    P = I.params_p2_stress(G=0.0, v=0.0)
    n = 10
    shape = (6, n, n)
    phi, mu = I.ic_voronoi(shape, seed=8, N=3, M=1)
    Q = np.array([[0.0, -1.0, 0.0], [1.0, 0.0, 0.0], [0.0, 0.0, 1.0]])  # (x, y) -> (-y, x)

    def rotf(a):  # new[x', y'] = old[x, y] with x' = n-1-y, y' = x: arrays are [c][z][y][x]
        return np.ascontiguousarray(np.rot90(a, k=1, axes=(3, 2)))

    o1 = oracle_mod.Oracle(shape, P)
    o1.init(phi, mu)
    o1.step(3)
    p1, m1 = o1.download()
    P2 = dict(P, aniso_R=np.einsum("abij,kj->abik", P["aniso_R"], Q))
    o2 = oracle_mod.Oracle(shape, P2)
    o2.init(rotf(phi), rotf(mu))
    o2.step(3)
    p2, m2 = o2.download()
    assert np.abs(rotf(p1) - p2).max() < 1e-13
    assert np.abs(rotf(m1) - m2).max() < 1e-13
    # and R is not symmetric in its use: the transposed rotation differs
    P3 = dict(P, aniso_R=np.einsum("abij,jk->abik", P["aniso_R"], Q))
    o3 = oracle_mod.Oracle(shape, P3)
    o3.init(rotf(phi), rotf(mu))
    o3.step(3)
    assert np.abs(rotf(p1) - o3.download()[0]).max() > 1e-8


def _sympy_pair_f(R, delta):
    """sympy's gradient and Hessian of the anisotropic pair energy
    f(q) = A(R q)^2 |q|^2, A(p) = 1 - delta (3 - 4 sum_i p_i^4 / |p|^4)
    (eq. 4 with reading B6), as numpy functions of q (3 x n arrays)."""
    import sympy as sp
    q = sp.symbols("q0:3", real=True)
    pv = sp.Matrix(R) * sp.Matrix(q)
    n2 = sum(c * c for c in pv)
    A = 1 - sp.Float(delta) * (3 - 4 * sum(c ** 4 for c in pv) / n2 ** 2)
    f = A ** 2 * n2
    grad = [sp.diff(f, q[i]) for i in range(3)]
    hess = [[sp.diff(f, q[i], q[j]) for j in range(3)] for i in range(3)]
    return sp.lambdify(q, grad, "numpy", cse=True), sp.lambdify(q, hess, "numpy", cse=True)


def _fields(Lbox, N, M):
    """Smooth periodic test fields (not on the simplex: r_a does not need it)
    with their gradients and Hessians, from sympy."""
    import sympy as sp
    X = sp.symbols("x y z", real=True)
    k = 2 * sp.pi / Lbox
    phis = [sp.Rational(1, 3) + sp.Rational(1, 5) * sp.sin(k * X[0] + a) * sp.cos(k * X[1] + 2 * a)
            + sp.Rational(1, 10) * sp.cos(k * X[2] + 0.5 * a) for a in range(N)]
    mus = [sp.Rational(1, 20) * sp.sin(k * (X[0] + X[1]) + i) * sp.cos(k * X[2]) for i in range(M)]
    fld = [sp.lambdify(X, p, "numpy") for p in phis]
    grd = [[sp.lambdify(X, sp.diff(p, X[d]), "numpy") for d in range(3)] for p in phis]
    hes = [[[sp.lambdify(X, sp.diff(p, X[d], X[e]), "numpy") for e in range(3)] for d in range(3)] for p in phis]
    fmu = [sp.lambdify(X, q, "numpy") for q in mus]
    return fld, grd, hes, fmu


def test_p2_sympy_variational_derivative(oracle_mod):
    """P7 for P2: r_a of the oracle converges at second order to the
    continuum variational derivative of eq. 3 with the anisotropic eq. 4.
    sympy differentiates the pair energy f(q) = A(R q)^2 |q|^2 (gradient g_f,
    Hessian H_f); with q_ab = u_a grad u_b - u_b grad u_a the chain rule gives
      d(eps a)/du_a = eps sum_b gamma_ab g_f(q_ab) . grad u_b,
      div d(eps a)/d grad u_a = -eps sum_b gamma_ab div(u_b g_f(q_ab)),
      div(u_b g_f) = grad u_b . g_f + u_b sum_{d,i} H_f[d,i] d_d q_i,
    and omega / psi of eqs. 5-6 add (16/pi^2) sum_b gamma_ab u_b / eps +
    sum gamma_abd u_b u_d / eps + psi_a h'(u_a).  A(q) is homogeneous of
    degree 0, so f is only C^1 where some q_ab vanishes (isolated points
    for smooth fields): the error is measured on seeded sample cells where
    every |q_ab| is at least 0.4 of its maximum."""
    P = I.params_p2_stress(G=0.0)
    N, M, eps = P["N"], P["M"], P["eps"]
    Lbox = 16.0
    pair = {(a, b): _sympy_pair_f(P["aniso_R"][a, b], P["aniso_delta"][a, b])
            for a in range(N) for b in range(N) if a != b}
    fld, grd, hes, fmu = _fields(Lbox, N, M)
    bc = lambda v, s: np.broadcast_to(np.asarray(v, dtype=float), s)
    errs = []
    rng = np.random.default_rng(1)
    T = P["T0"]
    for n in (16, 32, 64):
        dx = Lbox / n
        c = (np.arange(n) + 0.5) * dx
        Z, Y, X = np.meshgrid(c, c, c, indexing="ij")
        phi = np.stack([bc(f(X, Y, Z), X.shape) for f in fld]).astype(np.float64)
        mu = np.stack([bc(f(X, Y, Z), X.shape) for f in fmu]).astype(np.float64)
        o = oracle_mod.Oracle((n, n, n), dict(P, dx=dx))
        o.init(phi, mu)
        r = o.phi_rhs()
        idx = rng.integers(0, n, size=(6000, 3))
        xs, ys, zs = c[idx[:, 2]], c[idx[:, 1]], c[idx[:, 0]]
        s = xs.shape
        u = [bc(f(xs, ys, zs), s) for f in fld]
        g = [np.stack([bc(grd[a][d](xs, ys, zs), s) for d in range(3)]) for a in range(N)]
        h = [np.array([[bc(hes[a][d][e](xs, ys, zs), s) for e in range(3)] for d in range(3)]) for a in range(N)]
        m = [bc(f(xs, ys, zs), s) for f in fmu]
        qn = np.full(s, np.inf)
        for a in range(N):
            for b in range(a + 1, N):
                qq = np.sqrt(((u[a] * g[b] - u[b] * g[a]) ** 2).sum(0))
                qn = np.minimum(qn, qq / qq.max())
        keep = qn >= 0.4
        assert keep.mean() > 0.1
        err = scale = 0.0
        for a in range(N):
            ref = np.zeros(s)
            for b in range(N):
                if b == a:
                    continue
                gam = P["gamma"][a, b]
                q = u[a] * g[b] - u[b] * g[a]                    # q_ab, 3 x n
                dq = (g[a][:, None] * g[b][None, :] + u[a] * h[b]  # d_d q_i, [d][i]
                      - g[b][:, None] * g[a][None, :] - u[b] * h[a])
                gf = np.array(pair[(a, b)][0](*q))
                Hf = np.array(pair[(a, b)][1](*q))
                ref += eps * gam * (gf * g[b]).sum(0)                         # d(eps a)/du_a
                div = (g[b] * gf).sum(0) + u[b] * np.einsum("di...,di...->...", Hf, dq)
                ref += eps * gam * div                                         # - div d(eps a)/d grad u_a
                ref += 16.0 / np.pi ** 2 * gam * u[b] / eps
                for d2 in range(b + 1, N):
                    if d2 != a:
                        ref += P["gamma3"][a, b, d2] * u[b] * u[d2] / eps
            A = P["A0"][a] + P["A1"][a] * T
            B = P["B0"][a] + P["B1"][a] * T
            psi = sum(m[i] * A[i, j] * m[j] for i in range(M) for j in range(M)) + sum(B[i] * m[i] for i in range(M))
            psi = psi + P["C0"][a] + P["C1"][a] * T
            ref += psi * 6.0 * u[a] * (1.0 - u[a])
            got = r[a, idx[:, 0], idx[:, 1], idx[:, 2]]
            err = max(err, np.abs(got - ref)[keep].max())
            scale = max(scale, np.abs(ref).max())
        errs.append(err / scale)
    orders = np.log2(np.array(errs[:-1]) / np.array(errs[1:]))
    assert errs[-1] < 2e-3 and np.all(np.abs(orders - 2.0) < 0.3), (errs, orders)


@pytest.mark.parametrize("ic", ["R", "V"])
def test_p2_simplex_invariants(oracle_mod, ic):
    P = I.params_p2_stress()
    shape = (8, 10, 12)
    phi, mu = I.make_ic(ic, shape, seed=2, N=3, M=1)
    o = oracle_mod.Oracle(shape, P)
    o.init(phi, mu)
    for _ in range(4):
        o.step(1)
        p, _ = o.download()
        assert np.abs(p.sum(0) - 1.0).max() <= 8 * 2.2e-16
        assert p.min() >= 0.0
