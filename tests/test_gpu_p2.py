"""GPU parity of the P2 parameterisation (SURVEY §8(f) NEXT-4, P:L1199-1213;
pf_p2.cu): 3 phases, 1 chemical potential, anisotropic gradient energy
(reading B6), against the oracle on the same seeded inputs.  Bar as for P1
(north_star): relative L-inf <= 1e-12 after one step, <= 1e-9 after 1000.
-m gpu.
"""
import os

import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I

pytestmark = pytest.mark.gpu


def rel_linf(a, b):
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-300))


@pytest.fixture(scope="module")
def pfmod():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("GPU test without a CUDA device")
    from paper_conf_sc_0003hehshhkwnr19_b200 import build, pf
    build.build()
    return pf


@pytest.fixture(scope="module")
def omod():
    from oracle import oracle as O
    O.build()
    O.set_threads(min(16, os.cpu_count() or 1))
    return O


def run_pair(pfmod, omod, shape, P, phi, mu, chunks, bc=None):
    g = pfmod.PhaseField(shape, P, bc=bc)
    g.init_fields(phi, mu)
    o = omod.Oracle(shape, P, bc)
    o.init(phi, mu)
    out, done = [], 0
    for t in chunks:
        g.step(t - done)
        o.step(t - done)
        done = t
        gp, gm = g.download()
        op, om = o.download()
        out.append((t, rel_linf(gp, op), rel_linf(gm, om), g.state(), o.state()))
    g.close()
    return out


@pytest.mark.parametrize("kern", ["default", "mu_march", "phi_march", "naive"])
@pytest.mark.parametrize("pset", ["p2", "p2_stress", "p2_iso"])
@pytest.mark.parametrize("ic", ["R", "V"])
def test_p2_one_step_parity(pfmod, omod, pset, ic, kern, monkeypatch):
    """Default kernels (side-staged phi and mu; every face once, ragged tiles
    and z-chunks at this shape), the z-marching mu and phi kernels, and the
    one-thread-per-cell kernels."""
    monkeypatch.setenv("PF_P2_NAIVE", "1" if kern == "naive" else "0")
    monkeypatch.setenv("PF_P2_PHI", "march" if kern == "phi_march" else "side")
    monkeypatch.setenv("PF_P2_MU", "march" if kern == "mu_march" else "side")
    P = {"p2": I.params_p2(), "p2_stress": I.params_p2_stress(), "p2_iso": I.params_p2(aniso=0)}[pset]
    shape = (18, 21, 37)
    phi, mu = I.make_ic(ic, shape, seed=11, N=3, M=1)
    for t, ep, em, *_ in run_pair(pfmod, omod, shape, P, phi, mu, [1, 2]):
        assert ep <= 1e-12 and em <= 1e-12, (t, ep, em)


def test_p2_ds_window_parity(pfmod, omod):
    """DS boundaries (Dirichlet mu_inf != 0 at z_hi), frozen T with G v != 0,
    window shifts."""
    P = I.params_p2_stress(window_check=5, window_frac=0.5, v=0.05)
    shape = (32, 12, 20)
    phi, mu = I.ic_voronoi(shape, seed=5, N=3, M=1)
    res = run_pair(pfmod, omod, shape, P, phi, mu, [1, 40], bc=I.BC_DS)
    for t, ep, em, gs, os_ in res:
        assert gs == os_
        tol = 1e-12 if t == 1 else 1e-11
        assert ep <= tol and em <= tol, (t, ep, em)
    assert res[-1][3]["z_off"] > 0


def test_p2_ds_front_parity(pfmod, omod):
    """The benchmark's P2 directional-solidification recipe (params_p2_ds,
    ic_p2_front): grains under liquid, frozen gradient, DS boundaries, the
    window shifting at the first checks."""
    shape = (40, 16, 24)
    zf = 22
    P = I.params_p2_ds(zf, v=0.1)
    phi, mu = I.ic_p2_front(shape, seed=3, z_front=zf)
    res = run_pair(pfmod, omod, shape, P, phi, mu, [1, 60], bc=I.BC_DS)
    for t, ep, em, gs, os_ in res:
        assert gs == os_
        tol = 1e-12 if t == 1 else 1e-10
        assert ep <= tol and em <= tol, (t, ep, em)
    assert res[-1][3]["z_off"] > 0


def test_p2_1000_steps(pfmod, omod):
    P = I.params_p2_stress()
    shape = (16, 16, 16)
    phi, mu = I.ic_voronoi(shape, seed=6, N=3, M=1)
    for t, ep, em, *_ in run_pair(pfmod, omod, shape, P, phi, mu, [1, 100, 1000]):
        tol = 1e-12 if t == 1 else 1e-9
        assert ep <= tol and em <= tol, (t, ep, em)


def test_p2_liquid_index_not_hardcoded(pfmod, omod):
    """Any phase may be the liquid (compile-time L of the mu kernels)."""
    P = I.params_p2_stress()
    perm = [2, 1, 0]  # phase 0 plays the liquid
    Q = dict(P, liquid=0)
    for key in ("A0", "A1", "B0", "B1", "C0", "C1", "D"):
        Q[key] = P[key][perm]
    Q["gamma"] = P["gamma"][np.ix_(perm, perm)]
    Q["tau"] = P["tau"][np.ix_(perm, perm)]
    Q["gamma3"] = P["gamma3"][np.ix_(perm, perm, perm)]
    Q["aniso_delta"] = P["aniso_delta"][np.ix_(perm, perm)]
    Q["aniso_R"] = P["aniso_R"][np.ix_(perm, perm)]
    shape = (10, 12, 14)
    phi, mu = I.ic_voronoi(shape, seed=9, N=3, M=1)
    for t, ep, em, *_ in run_pair(pfmod, omod, shape, Q, phi, mu, [2]):
        assert ep <= 1e-12 and em <= 1e-12, (t, ep, em)


def test_p2_invariants_and_monitor(pfmod):
    P = I.params_p2()
    shape = (24, 24, 24)
    phi, mu = I.ic_voronoi(shape, seed=2, N=3, M=1)
    g = pfmod.PhaseField(shape, P)
    g.init_fields(phi, mu)
    g.set_monitors(5, 1e-13)
    g.step(50)
    err, mn = g.monitor()
    assert err <= 8 * 2.2e-16 and mn >= 0.0
    p, _ = g.download()
    assert p.shape == (3,) + shape


@pytest.mark.parametrize("kern", ["side", "side_hasync", "march", "naive"])
@pytest.mark.parametrize("pset", ["p2", "p2_stress", "p2_iso"])
def test_p2_specialised_equals_generic(pfmod, omod, pset, kern, monkeypatch):
    """The run-time specialised P2 sweeps (variant jit, the default: the
    bodies of pf_p2_dev.cuh on compile-time parameters, isotropic unrotated
    pairs as 2 q, unrotated pairs without rotation) give the generic
    kernels' bits (variant tuned), and the generic kernels meet the oracle
    bar on their own."""
    monkeypatch.setenv("PF_P2_NAIVE", "1" if kern == "naive" else "0")
    monkeypatch.setenv("PF_P2_PHI", "march" if kern == "march" else "side")
    monkeypatch.setenv("PF_P2_MU", "march" if kern == "march" else "side")
    # side_hasync: the specialised mu-sweep stages its halo ring by cp.async
    monkeypatch.setenv("PF_P2_HASYNC", "1" if kern == "side_hasync" else "0")
    P = {"p2": I.params_p2(), "p2_stress": I.params_p2_stress(), "p2_iso": I.params_p2(aniso=0)}[pset]
    shape = (18, 21, 37)
    phi, mu = I.ic_voronoi(shape, seed=13, N=3, M=1)
    outs = []
    for variant in ("jit", "tuned"):
        g = pfmod.PhaseField(shape, P)
        g.set_variant(variant)
        g.init_fields(phi, mu)
        g.step(3)
        outs.append(g.download())
        g.close()
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    o = omod.Oracle(shape, P)
    o.init(phi, mu)
    o.step(3)
    op, om = o.download()
    assert rel_linf(outs[1][0], op) <= 1e-12 and rel_linf(outs[1][1], om) <= 1e-12


@pytest.mark.parametrize("cfg", ["8x2", "8x1", "4x3", "4x4", "4x5", "4x6"])
def test_p2_side_tilings_bitwise(pfmod, monkeypatch, cfg):
    """The side-staged kernels' other tile heights / occupancies (PF_P2_SIDE)
    give the default's bits: each face flux is computed from the same two
    sides whichever thread evaluates it."""
    P = I.params_p2_stress()
    shape = (18, 21, 37)
    phi, mu = I.ic_voronoi(shape, seed=11, N=3, M=1)
    outs = []
    monkeypatch.setenv("PF_P2_PHI", "side")
    monkeypatch.setenv("PF_P2_MU", "side")
    for c in ("default", cfg):
        monkeypatch.setenv("PF_P2_SIDE", c)
        monkeypatch.setenv("PF_P2_SIDE_MU", c)
        g = pfmod.PhaseField(shape, P)
        g.init_fields(phi, mu)
        g.step(3)
        outs.append(g.download())
        g.close()
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])


@pytest.mark.parametrize("shape", [(1, 1, 1), (3, 5, 7), (5, 6, 62), (40, 70, 65)])
def test_p2_ragged_and_tiny_shapes(pfmod, omod, shape):
    P = I.params_p2_stress()
    phi, mu = I.ic_random(shape, seed=3, N=3, M=1)
    for t, ep, em, *_ in run_pair(pfmod, omod, shape, P, phi, mu, [2]):
        assert ep <= 1e-12 and em <= 1e-12, (shape, ep, em)


@pytest.mark.parametrize("pure", [2, 0])
def test_p2_pure_phase_fields(pfmod, omod, pure):
    """One phase everywhere (the liquid, or grain 0) with a random mu: the
    anisotropy sees q = 0 on every pair (grad f(0) = 0, the 0-branch of
    aniso_grad) and the anti-trapping guards fire on every face."""
    P = I.params_p2_stress()
    shape = (9, 14, 37)
    rng = np.random.default_rng(6)
    phi = np.zeros((3,) + shape)
    phi[pure] = 1.0
    mu = rng.uniform(-0.2, 0.2, size=(1,) + shape)
    res = run_pair(pfmod, omod, shape, P, phi, mu, [3])
    t, ep, em, *_ = res[-1]
    assert ep <= 1e-12 and em <= 1e-12, (ep, em)


def test_p2_autotune_and_tuning_knobs(pfmod, omod):
    """pf_autotune on a P2 context times every kernel choice of both sweeps
    (p2_* knobs) without touching the state; every choice keeps parity."""
    P = I.params_p2_stress()
    shape = (20, 24, 40)
    phi, mu = I.ic_voronoi(shape, seed=21, N=3, M=1)
    g = pfmod.PhaseField(shape, P)
    g.init_fields(phi, mu)
    rep = g.autotune(reps=3)
    assert g.state()["step"] == 0
    p0, m0 = g.download()
    assert np.array_equal(p0, phi) and np.array_equal(m0, mu)
    assert rep["phi"]["candidates"] > 10 and rep["mu"]["candidates"] > 10
    g.step(2)
    gp, gm = g.download()
    g.close()
    o = omod.Oracle(shape, P)
    o.init(phi, mu)
    o.step(2)
    op, om = o.download()
    assert rel_linf(gp, op) <= 1e-12 and rel_linf(gm, om) <= 1e-12
    for t in ({"p2_phi": 1, "p2_mu": 1}, {"p2_phi": 2, "p2_mu": 2},
              {"p2_phi_ty": 4, "p2_phi_minb": 3, "p2_mu_ty": 8, "p2_mu_minb": 1, "p2_phi_pd": 0, "p2_mu_pd": 4}):
        g = pfmod.PhaseField(shape, P)
        g.set_tuning(t)
        g.init_fields(phi, mu)
        g.step(2)
        gp, gm = g.download()
        g.close()
        assert rel_linf(gp, op) <= 1e-12 and rel_linf(gm, om) <= 1e-12, t
    with pytest.raises(pfmod.PFError):
        pfmod.PhaseField(shape, P).set_tuning({"p2_phi_ty": 4, "p2_phi_minb": 2})
