"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on
the same seeded inputs (pin P13).  -m gpu.

Bar (BASELINE.json north_star): relative L-inf per field, max|x - x_ref| /
max|x_ref| [A21], <= 1e-12 after one step and <= 1e-9 after 1000 steps.
"""
import os

import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I

pytestmark = pytest.mark.gpu

TOL_1 = 1e-12
TOL_1000 = 1e-9


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


def run_pair(pfmod, omod, shape, P, ic, steps, bc=None, seed=20191117, variant="jit", chunks=None, ic_kw=None):
    phi, mu = I.make_ic(ic, shape, seed=seed, **(ic_kw or {}))
    g = pfmod.PhaseField(shape, P, bc=bc)
    g.set_variant(variant)
    g.init_fields(phi, mu)
    o = omod.Oracle(shape, P, bc)
    o.init(phi, mu)
    out = []
    done = 0
    for target in (chunks or [steps]):
        g.step(target - done)
        o.step(target - done)
        done = target
        gp, gm = g.download()
        op, om = o.download()
        out.append((target, rel_linf(gp, op), rel_linf(gm, om), g.state(), o.state()))
    return out


@pytest.mark.parametrize("variant", ["jit", "tuned", "naive", "split"])
@pytest.mark.parametrize("pset", ["c4", "stress"])
@pytest.mark.parametrize("ic", ["R", "V", "L"])
def test_one_step_parity(pfmod, omod, variant, pset, ic):
    P = I.params_c4() if pset == "c4" else I.params_stress()
    shape = (20, 24, 40)  # several tiles and a ragged tail in x
    for t, ep, em, gs, os_ in run_pair(pfmod, omod, shape, P, ic, 1, variant=variant):
        assert ep <= TOL_1 and em <= TOL_1, (ep, em)


@pytest.mark.parametrize("variant", ["jit", "tuned", "jit_xsh"])
@pytest.mark.parametrize("shape", [(1, 1, 1), (3, 5, 7), (17, 9, 33), (8, 8, 130), (40, 70, 65), (5, 6, 62)])
def test_ragged_and_tiny_shapes(pfmod, omod, shape, variant, monkeypatch):
    P = I.params_stress()
    if variant == "jit_xsh":  # 31-cell tile rows: ragged at other widths (62 = 2 x 31)
        monkeypatch.setenv("PF_PHI_XSH", "1")
        variant = "jit"
    for t, ep, em, *_ in run_pair(pfmod, omod, shape, P, "R", 2, variant=variant):
        assert ep <= TOL_1 and em <= TOL_1, (shape, ep, em)


@pytest.mark.parametrize("liquid", [0, 2])
def test_liquid_index_not_hardcoded(pfmod, omod, liquid):
    """Any phase may be the liquid l of eq. 10: permute the C.4 set so that
    phase `liquid` plays the liquid, on both sides."""
    P = I.params_stress()
    perm = list(range(4))
    perm[3], perm[liquid] = perm[liquid], perm[3]
    Q = dict(P, liquid=liquid)
    for key in ("A0", "A1", "B0", "B1", "C0", "C1", "D"):
        Q[key] = P[key][perm]
    Q["gamma"] = P["gamma"][np.ix_(perm, perm)]
    Q["tau"] = P["tau"][np.ix_(perm, perm)]
    Q["gamma3"] = P["gamma3"][np.ix_(perm, perm, perm)]
    shape = (10, 12, 14)
    phi, mu = I.ic_voronoi(shape, seed=12)
    outs = {}
    for variant in ("jit", "tuned"):
        g = pfmod.PhaseField(shape, Q, liquid=liquid)
        g.set_variant(variant)
        g.init_fields(phi, mu)
        g.step(2)
        outs[variant] = g.download()
    o = omod.Oracle(shape, Q)
    o.init(phi, mu)
    o.step(2)
    op, om = o.download()
    for v, (gp, gm) in outs.items():
        assert rel_linf(gp, op) <= TOL_1 and rel_linf(gm, om) <= TOL_1, v


def test_config1_50_steps(pfmod, omod):
    """config 1: 32^3 periodic, 50 explicit steps, single device vs oracle."""
    P = I.params_c4()
    res = run_pair(pfmod, omod, (32, 32, 32), P, "V", 50, chunks=[1, 2, 5, 10, 50])
    for t, ep, em, *_ in res:
        tol = TOL_1 if t == 1 else 1e-11
        assert ep <= tol and em <= tol, (t, ep, em)


def test_1000_steps(pfmod, omod):
    P = I.params_stress()
    res = run_pair(pfmod, omod, (16, 16, 16), P, "V", 1000, chunks=[1, 100, 1000])
    for t, ep, em, *_ in res:
        tol = TOL_1 if t == 1 else TOL_1000
        assert ep <= tol and em <= tol, (t, ep, em)


def test_ds_window_parity(pfmod, omod):
    """config 2 structure at small size: DS BCs, frozen T, moving window."""
    P = I.params_c4("ds", window_check=5, window_frac=0.5, v=0.05)
    P["T0"] = I.ds_T0(20, P["G"])
    shape = (32, 12, 16)  # front above nz/2: the first check shifts
    res = run_pair(pfmod, omod, shape, P, "L", 60, bc=I.BC_DS, chunks=[1, 20, 60], ic_kw={"z_front": 20})
    for t, ep, em, gs, os_ in res:
        assert gs == os_, (gs, os_)
        tol = TOL_1 if t == 1 else 1e-11
        assert ep <= tol and em <= tol, (t, ep, em)
    assert res[-1][3]["z_off"] > 0


# DS boundaries with the stress set: mu_inf != 0, so the
# Dirichlet-mu ghost at z_hi [A15] differs from the interior from step 1 on
# (IC-R: mu ~ U(-0.1, 0.1)), A1 != 0 and G v != 0 (frozen T with a Q term),
# window inflow mu = mu_inf [A16].
@pytest.mark.parametrize("variant", ["jit", "tuned", "naive", "split"])
@pytest.mark.parametrize("window", [0, 1])
def test_ds_stress_one_step(pfmod, omod, variant, window):
    P = I.params_stress(window_check=window, window_frac=0.5)
    assert np.all(P["mu_inf"] != 0.0)
    shape = (20, 24, 40)
    res = run_pair(pfmod, omod, shape, P, "R", 2, bc=I.BC_DS, variant=variant, chunks=[1, 2])
    for t, ep, em, gs, os_ in res:
        assert gs == os_, (gs, os_)
        assert ep <= TOL_1 and em <= TOL_1, (t, ep, em)
    if window:
        assert res[0][3]["z_off"] > 0


def test_ds_stress_1000_steps(pfmod, omod):
    P = I.params_stress(window_check=50, window_frac=0.5)
    shape = (24, 16, 16)
    res = run_pair(pfmod, omod, shape, P, "V", 1000, bc=I.BC_DS, chunks=[1, 100, 1000])
    for t, ep, em, gs, os_ in res:
        assert gs == os_, (gs, os_)
        tol = TOL_1 if t == 1 else TOL_1000
        assert ep <= tol and em <= tol, (t, ep, em)
    assert res[-1][3]["z_off"] > 0


# Fluctuation term xi of eq. 7 (NEXT-3, Philox P:L669-676),
# reading B4: both sides draw the same Philox4x32-10 uniforms per cell/step.
@pytest.mark.parametrize("variant", ["jit", "tuned", "naive"])
@pytest.mark.parametrize("pset", ["c4", "stress"])
def test_fluctuation_parity(pfmod, omod, variant, pset):
    P = I.params_c4() if pset == "c4" else I.params_stress()
    P = dict(P, xi_amp=0.05, xi_seed=20191117)
    shape = (20, 24, 40)
    res = run_pair(pfmod, omod, shape, P, "V", 20, variant=variant, chunks=[1, 2, 20])
    for t, ep, em, *_ in res:
        tol = TOL_1 if t == 1 else 1e-11
        assert ep <= tol and em <= tol, (t, ep, em)


def test_fluctuation_ds_window_and_reproducible(pfmod, omod):
    """xi with the DS boundary conditions, frozen T and window shifts (global
    z counter = lattice index), 1000-step bar, and bitwise run-to-run."""
    P = I.params_c4("ds", window_check=5, window_frac=0.5, v=0.05, xi_amp=0.03, xi_seed=7)
    P["T0"] = I.ds_T0(20, P["G"])
    shape = (32, 12, 16)
    res = run_pair(pfmod, omod, shape, P, "L", 200, bc=I.BC_DS, chunks=[1, 200], ic_kw={"z_front": 20})
    for t, ep, em, gs, os_ in res:
        assert gs == os_
        tol = TOL_1 if t == 1 else TOL_1000
        assert ep <= tol and em <= tol, (t, ep, em)
    phi, mu = I.ic_lamellar(shape, seed=20191117, z_front=20)
    outs = []
    for _ in range(2):
        g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
        g.init_fields(phi, mu)
        g.step(30)
        outs.append(g.download())
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])


def test_step_phi_only(pfmod, omod):
    P = I.params_stress()
    shape = (12, 10, 14)
    phi, mu = I.ic_voronoi(shape, seed=4)
    g = pfmod.PhaseField(shape, P)
    g.init_fields(phi, mu)
    g.step_phi_only()
    o = omod.Oracle(shape, P)
    o.init(phi, mu)
    o.step_phi_only()
    gp, gm = g.download()
    op, om = o.download()
    assert rel_linf(gp, op) <= TOL_1 and np.array_equal(gm, mu)


def test_bitwise_reproducible_and_variants(pfmod):
    P = I.params_stress()
    shape = (24, 20, 36)
    phi, mu = I.ic_voronoi(shape, seed=5)
    outs = []
    for _ in range(2):
        g = pfmod.PhaseField(shape, P)
        g.init_fields(phi, mu)
        g.step(7)
        outs.append(g.download())
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])


def test_forced_exchange_path_bitwise(pfmod, monkeypatch):
    """The pack / exchange / unpack path (used across ranks) gives bitwise
    the same ghosts as the local periodic fill."""
    P = I.params_stress()
    shape = (10, 12, 14)
    phi, mu = I.ic_voronoi(shape, seed=6)
    g = pfmod.PhaseField(shape, P)
    g.init_fields(phi, mu)
    g.step(3)
    ref = g.download()
    monkeypatch.setenv("PF_FORCE_EXCHANGE", "1")
    h = pfmod.PhaseField(shape, P)
    h.init_fields(phi, mu)
    h.step(3)
    got = h.download()
    assert np.array_equal(ref[0], got[0]) and np.array_equal(ref[1], got[1])


@pytest.mark.parametrize("bc", ["periodic", "ds"])
def test_nccl_self_exchange_bitwise(pfmod, monkeypatch, bc):
    """The world > 1 code path on one GPU: PF_FORCE_EXCHANGE=nccl gives the
    context a 1-rank NCCL communicator, so the halo exchange of every
    periodic dimension goes through pack -> ncclSend/ncclRecv to itself ->
    unpack (on the comm stream, overlapped with the interior mu tiles), and
    the window / monitor reductions through ncclAllReduce.  Bitwise equal to
    the local ghost fill; window shifts included for the DS case."""
    if bc == "periodic":
        P, B, shape = I.params_stress(), None, (40, 20, 70)
        phi, mu = I.ic_voronoi(shape, seed=8)
    else:
        P = I.params_c4("ds", window_check=2, window_frac=0.3)
        B, shape = I.BC_DS, (24, 20, 40)
        phi, mu = I.ic_lamellar(shape, seed=3, z_front=10)
    outs = []
    # z faces go as whole planes in place (zero copy) unless PF_ZC_EXCHANGE=0
    for force, zc in (("0", "1"), ("nccl", "1"), ("nccl", "0")):
        monkeypatch.setenv("PF_FORCE_EXCHANGE", force)
        monkeypatch.setenv("PF_ZC_EXCHANGE", zc)
        g = pfmod.PhaseField(shape, P, bc=B)
        g.init_fields(phi, mu)
        g.step(6)
        rep = g.autotune(mask=pfmod.PF_MU, passes=1, reps=2) if force == "nccl" else None
        g.step(4)
        outs.append((g.download(), g.state(), g.monitor(), g.front_height()))
        g.close()
    (a, sa, ma, ha) = outs[0]
    for (b, sb, mb, hb) in outs[1:]:
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
        assert sa == sb and ha == hb and np.array_equal(ma, mb)
    if bc == "ds":
        assert sa["z_off"] > 0  # the window shifted (collective front height)


@pytest.mark.parametrize("case", ["ds_window", "stress_xi", "nccl_periodic"])
def test_graph_steps_bitwise(pfmod, monkeypatch, case):
    """pf_step replays runs of steps between window checks as CUDA graphs
    (S§8(d) D.7), the sweeps reading each step's T base and step index from
    device memory: bitwise equal to launching every step (PF_GRAPH=0) --
    frozen temperature moving with v t, window shifts, the fluctuation
    counter (step) and the NCCL exchange inside the captured graph."""
    if case == "ds_window":
        P = I.params_c4("ds", window_check=7, window_frac=0.3)
        B, shape = I.BC_DS, (24, 20, 40)
        phi, mu = I.ic_lamellar(shape, seed=3, z_front=10)
    else:
        P = I.params_stress(xi_amp=0.02, xi_seed=7) if case == "stress_xi" else I.params_stress()
        B, shape = None, (20, 24, 40)
        phi, mu = I.ic_voronoi(shape, seed=5)
    if case == "nccl_periodic":
        monkeypatch.setenv("PF_FORCE_EXCHANGE", "nccl")
    outs = []
    for gr in ("0", "1"):
        monkeypatch.setenv("PF_GRAPH", gr)
        g = pfmod.PhaseField(shape, P, bc=B)
        g.init_fields(phi, mu)
        for n in (1, 5, 30, 2, 70):  # runs of several lengths: new and cached graphs, both buffer parities
            g.step(n)
        outs.append((g.download(), g.state()))
        g.close()
    (a, sa), (b, sb) = outs
    assert sa == sb
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    if case == "ds_window":
        assert sa["z_off"] > 0


def test_graph_steps_profiled(pfmod, monkeypatch):
    """pf_profile timing with graph steps: the per-kernel events are event
    nodes of the captured graph, collected after each replay; launch counts
    are those of the direct steps."""
    P = I.params_c4("ds", window_check=5, window_frac=0.5)
    shape = (24, 20, 40)
    phi, mu = I.ic_lamellar(shape, seed=3, z_front=6)
    res = {}
    for gr in ("0", "1"):
        monkeypatch.setenv("PF_GRAPH", gr)
        g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
        g.init_fields(phi, mu)
        g.profile(True)
        g.step(10)
        g.profile(True)  # reset counters, keep the graphs
        g.step(20)
        res[gr] = (g.profile_read(), g.download())
        g.close()
    (pa, a), (pb, b) = res["0"], res["1"]
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    for k in ("phi_sweep", "mu_sweep"):
        assert pa[k][1] == pb[k][1] == 20, (k, pa[k], pb[k])
        assert pb[k][0] > 0.0
    assert pa["ghost"][1] == pb["ghost"][1]


@pytest.mark.parametrize("variant", ["jit", "tuned"])
def test_overlapped_exchange_bitwise(pfmod, monkeypatch, variant):
    """Interior/shell split of the mu-sweep with the phi exchange on a second
    stream and the mu exchange overlapping the next phi-sweep,
    and (no exchange) the local mu ghost fill on the side stream: bitwise
    equal to the serial schedule and to the local ghost fill."""
    P = I.params_stress()
    shape = (70, 20, 100)  # 4 x-tiles, 5 y-tiles, 3 z-chunks: non-empty interior
    phi, mu = I.ic_voronoi(shape, seed=8)
    outs = []
    for force, overlap in (("0", "0"), ("0", "1"), ("1", "0"), ("1", "1")):
        monkeypatch.setenv("PF_FORCE_EXCHANGE", force)
        monkeypatch.setenv("PF_OVERLAP", overlap)
        g = pfmod.PhaseField(shape, P)
        g.set_variant(variant)
        g.init_fields(phi, mu)
        g.step(4)
        outs.append(g.download())
    for o in outs[1:]:
        assert np.array_equal(outs[0][0], o[0]) and np.array_equal(outs[0][1], o[1])


def test_translation_invariance_bitwise(pfmod):
    P = I.params_stress(G=0.0, v=0.0)
    shape = (16, 12, 20)
    phi, mu = I.ic_voronoi(shape, seed=7)
    roll = lambda a: np.roll(a, (3, 2, 5), axis=(1, 2, 3))
    g = pfmod.PhaseField(shape, P)
    g.init_fields(phi, mu)
    g.step(4)
    a = g.download()
    h = pfmod.PhaseField(shape, P)
    h.init_fields(roll(phi), roll(mu))
    h.step(4)
    b = h.download()
    assert np.array_equal(roll(a[0]), b[0]) and np.array_equal(roll(a[1]), b[1])


def test_monitors_front_and_shift(pfmod, omod):
    P = I.params_c4("ds")
    shape = (24, 8, 12)
    phi, mu = I.ic_lamellar(shape, seed=3, z_front=10)
    g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
    g.init_fields(phi, mu)
    o = omod.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    assert g.front_height() == o.front_height()
    e, mn = g.monitor()
    assert e == np.abs(phi.sum(0) - 1).max() and mn == phi.min()
    g.shift_window(4)
    o.shift_window(4)
    gp, gm = g.download()
    op, om = o.download()
    assert np.array_equal(gp, op) and np.array_equal(gm, om)
    assert g.state() == o.state()


def test_rejects_bad_input(pfmod):
    P = I.params_c4()
    shape = (4, 4, 4)
    g = pfmod.PhaseField(shape, P)
    phi, mu = I.ic_random(shape)
    phi[0, 0, 0, 0] += 1e-9
    with pytest.raises(pfmod.PFError):
        g.init_fields(phi, mu)
    with pytest.raises(pfmod.PFError):
        g.set_params(dict(P, dt=0.2))  # above the explicit stability bound
    with pytest.raises(pfmod.PFError):
        g.step(1)  # no fields yet


def test_e2e_pinned_roundtrip(pfmod):
    import torch
    P = I.params_c4()
    shape = (8, 8, 8)
    phi, mu = I.ic_random(shape)
    g = pfmod.PhaseField(shape, P)
    tp = torch.from_numpy(phi).pin_memory()
    tm = torch.from_numpy(mu).pin_memory()
    g.init_fields(tp, tm)
    op = torch.empty_like(tp).pin_memory()
    om = torch.empty_like(tm).pin_memory()
    g.download(out=(op, om))
    assert np.array_equal(op.numpy(), phi) and np.array_equal(om.numpy(), mu)


def test_split_variant_bitwise_equals_full(pfmod):
    """The split kernels (staggered fluxes through a global array, the
    paper's "split" variant) evaluate the same face and cell arithmetic in
    the same order as the full (naive) kernels: bitwise equal, DS + window."""
    P = I.params_stress(window_check=4, window_frac=0.5, xi_amp=0.02, xi_seed=5)
    shape = (24, 18, 37)
    phi, mu = I.ic_lamellar(shape, seed=4, z_front=14, mu_inf=tuple(P["mu_inf"]))
    outs = []
    for v in ("naive", "split"):
        g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
        g.set_variant(v)
        g.init_fields(phi, mu)
        g.step(12)
        outs.append((g.download(), g.state()))
        g.close()
    assert outs[0][1] == outs[1][1] and outs[0][1]["z_off"] > 0
    assert np.array_equal(outs[0][0][0], outs[1][0][0]) and np.array_equal(outs[0][0][1], outs[1][0][1])


@pytest.mark.parametrize("variant", ["jit", "tuned", "naive", "split"])
@pytest.mark.parametrize("pure", [3, 0])
def test_pure_phase_fields(pfmod, omod, variant, pure):
    """Degenerate fields: one phase everywhere (the liquid, or solid 0) with a
    random mu.  Every gradient term and the anti-trapping current vanish
    (the exact-zero guards [A11]); phi feels only the obstacle and driving
    forces at the simplex corner, which the projection absorbs, and mu
    evolves by diffusion alone -- as in the oracle."""
    P = I.params_stress()
    shape = (9, 14, 37)
    rng = np.random.default_rng(5)
    phi = np.zeros((4,) + shape)
    phi[pure] = 1.0
    mu = rng.uniform(-0.2, 0.2, size=(2,) + shape)
    g = pfmod.PhaseField(shape, P)
    g.set_variant(variant)
    g.init_fields(phi, mu)
    o = omod.Oracle(shape, P)
    o.init(phi, mu)
    g.step(3)
    o.step(3)
    gp, gm = g.download()
    op, om = o.download()
    assert rel_linf(gp, op) <= TOL_1 and rel_linf(gm, om) <= TOL_1
    assert np.abs(gp.sum(axis=0) - 1.0).max() <= 8 * 2.2e-16 and gp.min() >= 0.0
