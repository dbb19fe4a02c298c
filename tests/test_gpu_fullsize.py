"""Parity at the full BASELINE size, in the launch configuration bench.py
times (256^3 block, DS boundary conditions, frozen T, C.4 parameters, IC-L,
specialised kernels), on sampled cells that the oracle computes one by one.

One step of the method updates a cell from a neighbourhood of radius 2 (the
mu-sweep reads phi_dst at radius 1, which reads phi_src at radius 1), so the
oracle stepped on a 5^3 (or boundary-aligned 5-deep) sub-block extracted
around a sample reproduces that cell exactly; the frozen temperature of the
sub-block is placed with z_off = its global origin (reading A13).  Properties
that hold at any size (simplex invariants, bitwise reproducibility, periodic
translation) cover the long runs.  -m gpu."""
import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I

pytestmark = pytest.mark.gpu

NFULL = 256


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
    return O


ZF = NFULL // 2 + 2  # bench.py: the growing front starts two planes above the window threshold


@pytest.fixture(scope="module")
def bench_case(pfmod):
    """The bench.py workload: 256^3, DS BCs, C.4 parameters with the growing
    front (inputs.DS_BENCH), IC-L."""
    n = NFULL
    P = I.params_ds_growth(ZF, window_check=10, window_frac=0.5, **I.DS_BENCH)
    phi, mu = I.ic_lamellar((n, n, n), seed=20191117, z_front=ZF)
    g = pfmod.PhaseField((n, n, n), P, bc=I.BC_DS)
    g.init_fields(phi, mu)
    g.step(1)
    gp, gm = g.download()
    return P, phi, mu, gp, gm, g


def _sub_block(arr, zs, ys, xs):
    """arr[:, zs][:, :, ys][..., xs] with periodic x, y indices."""
    return arr[:, zs][:, :, ys % arr.shape[2]][:, :, :, xs % arr.shape[3]]


def test_sampled_cells_match_oracle(omod, bench_case):
    P, phi, mu, gp, gm, _ = bench_case
    n = NFULL
    rng = np.random.default_rng(20191117)
    # samples: random interior, around the front, and at the z boundaries
    zs = list(rng.integers(2, n - 2, 120)) + list(rng.integers(ZF - 8, ZF + 8, 60)) + [0, 1, 2, n - 3, n - 2, n - 1]
    ys = rng.integers(0, n, len(zs))
    xs = rng.integers(0, n, len(zs))
    Pq = dict(P, window_check=0)
    errp, errm = 0.0, 0.0
    scale_p, scale_m = np.abs(gp).max(), np.abs(gm).max()
    for z, y, x in zip(zs, ys, xs):
        if z < 2:
            z0, bc = 0, {"lo": ("periodic", "periodic", "neumann"), "hi": ("periodic", "periodic", "neumann")}
        elif z > n - 3:
            z0, bc = n - 5, {"lo": ("periodic", "periodic", "neumann"), "hi": ("periodic", "periodic", "dirichlet_mu")}
        else:
            z0, bc = z - 2, I.BC_PERIODIC  # sub-block faces are 2 cells away: their BC never reaches the centre
        zr = np.arange(z0, z0 + 5)
        yr = np.arange(y - 2, y + 3)
        xr = np.arange(x - 2, x + 3)
        sp = _sub_block(phi, zr, yr, xr).copy()
        sm = _sub_block(mu, zr, yr, xr).copy()
        o = omod.Oracle((5, 5, 5), Pq, bc)
        o.init(sp, sm)
        o.set_state(step=0, z_off=z0)
        o.step(1)
        op, om = o.download()
        k = z - z0
        errp = max(errp, np.abs(op[:, k, 2, 2] - gp[:, z, y, x]).max())
        errm = max(errm, np.abs(om[:, k, 2, 2] - gm[:, z, y, x]).max())
    assert errp / scale_p <= 1e-12 and errm / scale_m <= 1e-12, (errp / scale_p, errm / scale_m)


def test_fullsize_invariants_and_reproducibility(pfmod, bench_case):
    """Sum phi = 1, phi >= 0 after 1 and 50 more steps (window checks
    included) and bitwise run-to-run reproducibility at 256^3; the second run
    is auto-tuned first, as bench.py does (pf_autotune), so the tuning the
    bench times gives the same bits as the default one the samples check."""
    P, phi, mu, gp, gm, g = bench_case
    assert np.abs(gp.sum(0) - 1.0).max() <= 8 * 2.2e-16 and gp.min() >= 0.0
    g.step(50)
    e, mn = g.monitor()
    assert e <= 8 * 2.2e-16 and mn >= 0.0
    a = g.download()
    h = pfmod.PhaseField((NFULL,) * 3, P, bc=I.BC_DS)
    h.init_fields(phi, mu)
    h.autotune(passes=1, reps=3)
    h.step(51)
    b = h.download()
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert g.state() == h.state()


def test_fullsize_periodic_translation(pfmod):
    """Periodic 128^3 stress-set run: a translated input gives the bitwise
    translated output after 20 steps (property valid at any size)."""
    n = 128
    P = I.params_stress(G=0.0, v=0.0)
    phi, mu = I.ic_voronoi((n, n, n), seed=3, nseeds=24)
    g = pfmod.PhaseField((n, n, n), P)
    g.init_fields(phi, mu)
    g.step(20)
    a = g.download()
    roll = lambda q: np.roll(q, (17, 5, 40), axis=(1, 2, 3))
    h = pfmod.PhaseField((n, n, n), P)
    h.init_fields(roll(phi), roll(mu))
    h.step(20)
    b = h.download()
    assert np.array_equal(roll(a[0]), b[0]) and np.array_equal(roll(a[1]), b[1])


def test_p2_fullsize_sampled_cells(pfmod, omod):
    """P2 (NEXT-4) in the configuration bench.py times: 256^3 periodic,
    params_p2, IC-V; one step on the GPU, sampled cells against the oracle on
    5^3 periodic sub-blocks (the 19-point phi stencil still has radius 1,
    so a step reads radius 2)."""
    n = NFULL
    P = I.params_p2()
    phi, mu = I.ic_voronoi((n, n, n), seed=20191117, N=3, M=1)
    g = pfmod.PhaseField((n, n, n), P)
    g.init_fields(phi, mu)
    g.step(1)
    gp, gm = g.download()
    g.close()
    assert np.abs(gp.sum(0) - 1.0).max() <= 8 * 2.2e-16 and gp.min() >= 0.0
    rng = np.random.default_rng(7)
    # samples in interfaces (where every term is active) and anywhere
    mixed = np.argwhere(phi.max(0) < 0.99)
    pick = mixed[rng.integers(0, len(mixed), 120)]
    anyc = rng.integers(0, n, (40, 3))
    errp = errm = 0.0
    scale_p, scale_m = np.abs(gp).max(), np.abs(gm).max()
    for z, y, x in list(pick) + list(anyc):
        # (periodic in z as well: wrap the sub-block's planes)
        zr, yr, xr = np.arange(z - 2, z + 3) % n, np.arange(y - 2, y + 3), np.arange(x - 2, x + 3)
        sp = _sub_block(phi, zr, yr, xr).copy()
        sm = _sub_block(mu, zr, yr, xr).copy()
        o = omod.Oracle((5, 5, 5), P)
        o.init(sp, sm)
        o.step(1)
        op, om = o.download()
        errp = max(errp, np.abs(op[:, 2, 2, 2] - gp[:, z, y, x]).max())
        errm = max(errm, np.abs(om[:, 2, 2, 2] - gm[:, z, y, x]).max())
    assert errp / scale_p <= 1e-12 and errm / scale_m <= 1e-12, (errp / scale_p, errm / scale_m)


def test_stress_fullsize_sampled_cells(pfmod, omod):
    """Parameter set S (every general expression: unequal gamma, off-diagonal
    chi and D, A1 != 0, G v != 0) at the full 256^3 size, IC-V, periodic:
    one step, sampled cells against oracle sub-blocks (radius 2, z_off at the
    sub-block origin for the frozen temperature)."""
    n = NFULL
    P = I.params_stress()
    phi, mu = I.ic_voronoi((n, n, n), seed=20191119)
    g = pfmod.PhaseField((n, n, n), P)
    g.init_fields(phi, mu)
    g.step(1)
    gp, gm = g.download()
    g.close()
    rng = np.random.default_rng(7)
    # z kept 2 planes from the (periodic) z ends: with G v != 0 the frozen
    # temperature jumps across the periodic z boundary, which a sub-block
    # placed by z_off cannot reproduce
    zs, ys, xs = rng.integers(2, n - 2, 80), rng.integers(0, n, 80), rng.integers(0, n, 80)
    errp = errm = 0.0
    for z, y, x in zip(zs, ys, xs):
        zr, yr, xr = np.arange(z - 2, z + 3), np.arange(y - 2, y + 3), np.arange(x - 2, x + 3)
        o = omod.Oracle((5, 5, 5), dict(P, window_check=0), I.BC_PERIODIC)
        o.init(_sub_block(phi, zr, yr, xr).copy(), _sub_block(mu, zr, yr, xr).copy())
        o.set_state(step=0, z_off=int(z) - 2)
        o.step(1)
        op, om = o.download()
        errp = max(errp, np.abs(op[:, 2, 2, 2] - gp[:, z, y, x]).max())
        errm = max(errm, np.abs(om[:, 2, 2, 2] - gm[:, z, y, x]).max())
    assert errp / np.abs(gp).max() <= 1e-12 and errm / np.abs(gm).max() <= 1e-12, (errp, errm)


def test_fullsize_tunings_bitwise(pfmod, bench_case):
    """The bench launch configuration against its neighbours at full size:
    the halo ring loaded instead of cp.async-staged (mu_hasync 0, with the
    L1 prefetch) and the anti-trapping skip (mu_atskip 1) give the default's
    bits after one step of the bench workload."""
    P, phi, mu, gp, gm, _ = bench_case
    n = NFULL
    for t in ({"mu_hasync": 0, "mu_halo_l1": 1}, {"mu_atskip": 1}):
        g = pfmod.PhaseField((n, n, n), P, bc=I.BC_DS)
        g.set_tuning(t)
        g.init_fields(phi, mu)
        g.step(1)
        p, m = g.download()
        g.close()
        assert np.array_equal(p, gp) and np.array_equal(m, gm), t
