"""Auto-tuning of the specialised sweeps (S§8(f) NEXT-2; "an
auto-tuning mechanism can then test and optimize different mappings",
P:L808-865 per-kernel tuning): every tuning computes the same step, the
tuner leaves the state untouched and keeps the fastest setting.  -m gpu.

The bar is the parity bar of test_gpu_parity.py (<= 1e-12 after one step
against the oracle) for tuned corners, and bitwise equality between tunings:
the arithmetic per cell does not depend on the thread-to-cell mapping, the
occupancy or the schedule transformations (each face flux is evaluated on
the same two operands whichever thread computes it).
"""
import os

import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I

pytestmark = pytest.mark.gpu

TOL_1 = 1e-12

# corners of the search space of pf_autotune (tile shapes, occupancy,
# z-chunks, schedule transformations)
# one tile row per thread on the 32 x 4 tile (the rows-per-thread knob
# mu_rpt defaults to 2 on a 32 x 8 tile); knobs that need it start from here
R1 = {"mu_rpt": 1, "mu_ty": 4, "mu_minb": 3}
CORNERS = [
    {},
    {"phi_ty": 16, "phi_minb": 1, "phi_faces6": 0, "phi_unroll": 4, "phi_prefetch": 2, "phi_pfd": 3,
     "phi_xghost": 1},
    {"phi_ty": 8, "phi_minb": 2, "phi_zc": 5, "phi_faces6": 0, "phi_prefetch": 0},
    dict(R1, **{"mu_ty": 8, "mu_tx": 16, "mu_minb": 4, "mu_rpf": 0, "mu_halo_l1": 0, "mu_fxreg": 0, "mu_prefetch": 0}),
    dict(R1, **{"mu_ty": 3, "mu_minb": 5, "mu_zc": 7, "mu_pfd": 3, "mu_prefetch": 2}),
    {"mu_ty": 6, "mu_minb": 2, "mu_zc": 24, "phi_zc": 32, "phi_unroll": 3, "phi_xghost": 1},
    dict(R1, **{"mu_ldhint": 1, "mu_qreg": 1, "phi_xghost": 1}),
    dict(R1, **{"mu_ldhint": 2, "mu_tx": 16, "mu_ty": 4, "mu_minb": 4}),
    dict(R1, **{"mu_hpipe": 1, "phi_zrec": 1}),
    {"phi_xsh": 1},
    {"phi_xsh": 1, "phi_ty": 8, "phi_minb": 2, "phi_xghost": 1, "phi_zc": 7},
    dict(R1, **{"mu_hpipe": 1, "mu_rpf": 0, "mu_ty": 5, "mu_minb": 3, "phi_zrec": 1, "phi_faces6": 0}),
    # clusters stacked in y: 6 tiles of 4 rows (the last one ragged) in
    # clusters of 2; clusters of 4 do not tile them (plain kernels)
    dict(R1, mu_cly=2),
    dict(R1, mu_cly=4),
    dict(R1, **{"mu_cly": 2, "mu_ty": 3, "mu_minb": 5}),
    dict(R1, **{"mu_cly": 2, "mu_qreg": 1, "mu_fxreg": 0, "mu_hpipe": 1}),
    # tile rows rotated over the warps (plain and cluster kernels)
    dict(R1, mu_rot=1),
    dict(R1, **{"mu_rot": 1, "mu_ty": 5, "mu_minb": 3, "mu_cly": 2}),
    # two tile rows per thread (3 / 4 ragged tiles in y), one row per thread
    {"mu_rpt": 2, "mu_ty": 8, "mu_minb": 2, "mu_zc": 5, "mu_prefetch": 0, "mu_halo_l1": 0, "mu_ldhint": 1},
    {"mu_rpt": 2, "mu_ty": 6, "mu_minb": 3, "mu_rpf": 0, "mu_fxreg": 0, "mu_prefetch": 2},
    R1,
    # phi-sweep with two rows per thread (21 rows: the last pair's upper row is the ghost row)
    {"phi_rpt": 2, "phi_ty": 8, "phi_minb": 3},
    {"phi_rpt": 2, "phi_ty": 4, "phi_minb": 6, "phi_zc": 7, "phi_prefetch": 2, "phi_xghost": 1},
    # the carried side of the two-rows mu-sweep in tensor memory (TMEM)
    {"mu_tmem": 1, "mu_rpf": 0, "mu_minb": 3},
    {"mu_tmem": 1, "mu_zc": 7, "mu_ty": 6, "mu_minb": 3},
    # persistent launches: balanced tile-plane shares, segments crossing tile columns
    {"mu_pers": 1, "phi_pers": 1},
    {"mu_pers": 1, "mu_ty": 6, "mu_minb": 3, "phi_pers": 1, "phi_ty": 8, "phi_minb": 2, "phi_xsh": 1},
    # the halo ring's z column carried in shared memory (alone, ragged
    # chunks, with persistent shares and with the TMEM side)
    {"mu_hcar": 1},
    {"mu_hcar": 1, "mu_zc": 7, "mu_ty": 6, "mu_minb": 3, "mu_rpf": 0},
    {"mu_hcar": 1, "mu_pers": 1, "mu_ty": 10, "mu_minb": 2},
    {"mu_hcar": 1, "mu_tmem": 1, "mu_halo_l1": 0},
    # own cd_x by warp shuffles, L1 policies
    {"mu_xshfl": 1},
    {"mu_xshfl": 1, "mu_hcar": 1, "mu_ldhint": 3, "mu_ty": 6, "mu_minb": 3, "mu_zc": 5},
    # warp-uniform skip of the anti-trapping current where it is exactly 0
    {"mu_atskip": 1},
    dict(R1, mu_atskip=1),
    # the halo ring staged one plane ahead by cp.async (alone, ragged chunks /
    # tiles, without the L1 prefetch, with persistent shares, with shuffles)
    {"mu_hasync": 1},
    {"mu_hasync": 1, "mu_zc": 7, "mu_ty": 6, "mu_minb": 3, "mu_rpf": 0, "mu_halo_l1": 0},
    {"mu_hasync": 1, "mu_pers": 1, "mu_ty": 10, "mu_minb": 2},
    {"mu_hasync": 1, "mu_xshfl": 1, "mu_zc": 5},
    {"mu_hasync": 2, "mu_halo_l1": 0},
    {"mu_hasync": 2, "mu_zc": 7, "mu_ty": 6, "mu_minb": 3},
    {"mu_hasync": 2, "mu_pers": 1, "mu_ty": 10, "mu_minb": 2, "mu_xshfl": 1},
]


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


def gpu_run(pfmod, shape, P, phi, mu, steps, tuning=None, bc=None):
    g = pfmod.PhaseField(shape, P, bc=bc)
    if tuning:
        g.set_tuning(tuning)
    g.init_fields(phi, mu)
    g.step(steps)
    out = g.download()
    g.close()
    return out


@pytest.mark.parametrize("pset", ["c4", "stress"])
def test_tuning_corners_bitwise_and_parity(pfmod, omod, pset):
    P = I.params_c4("ds") if pset == "c4" else I.params_stress()
    bc = I.BC_DS if pset == "c4" else None
    shape = (23, 21, 45)  # ragged in every tile dimension of every corner
    phi, mu = I.make_ic("L" if pset == "c4" else "R", shape, seed=7)
    o = omod.Oracle(shape, P, bc)
    o.init(phi, mu)
    o.step(1)
    op, om = o.download()
    ref3 = None
    for c in CORNERS:
        gp, gm = gpu_run(pfmod, shape, P, phi, mu, 1, c, bc)
        assert rel_linf(gp, op) <= TOL_1 and rel_linf(gm, om) <= TOL_1, c
        g3 = gpu_run(pfmod, shape, P, phi, mu, 3, c, bc)
        if ref3 is None:
            ref3 = g3
        assert np.array_equal(g3[0], ref3[0]) and np.array_equal(g3[1], ref3[1]), c


def test_set_tuning_rejects_out_of_range(pfmod):
    shape = (8, 8, 32)
    g = pfmod.PhaseField(shape, I.params_c4())
    with pytest.raises(pfmod.PFError):
        g.set_tuning({"mu_ty": 9})
    with pytest.raises(pfmod.PFError):
        g.set_tuning({"phi_ty": 16, "phi_minb": 8})
    with pytest.raises(pfmod.PFError):
        g.set_tuning({"mu_ty": 5})  # odd tile height with two rows per thread
    with pytest.raises(pfmod.PFError):
        g.set_tuning({"mu_hcar": 1, "mu_hpipe": 1})
    g.set_tuning({"mu_ty": 6})
    assert g.tuning()["mu_ty"] == 6
    g.set_tuning(dict(R1, mu_ty=5))
    assert g.tuning()["mu_ty"] == 5


def test_autotune_keeps_state_and_result(pfmod):
    """pf_autotune on a DS block: state (fields, step, z_off) unchanged, the
    chosen tuning is valid and reported, and the run continues bitwise as
    with the default tuning."""
    P = I.params_c4("ds")
    shape = (48, 64, 64)
    phi, mu = I.make_ic("L", shape, seed=3)
    g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
    g.init_fields(phi, mu)
    g.step(2)
    before = g.download()
    st = g.state()
    rep = g.autotune(passes=1, reps=3)
    assert g.state() == st
    after = g.download()
    assert np.array_equal(before[0], after[0]) and np.array_equal(before[1], after[1])
    assert rep["best"] == g.tuning()
    assert pfmod.tuning_check(rep["best"]) == "ok"
    for k in ("phi", "mu"):
        assert rep[k]["best_ms"] <= rep[k]["start_ms"] and rep[k]["candidates"] > 5
    assert all((c["ms"] is None) == bool(c["error"]) for c in rep["tried"])
    assert sum(c["ms"] is not None for c in rep["tried"]) >= 10
    g.step(3)
    tuned = g.download()
    g.close()
    ref = gpu_run(pfmod, shape, P, phi, mu, 5, None, I.BC_DS)
    assert np.array_equal(tuned[0], ref[0]) and np.array_equal(tuned[1], ref[1])


def test_autotune_requires_fields_and_jit(pfmod):
    g = pfmod.PhaseField((8, 8, 32), I.params_c4())
    with pytest.raises(pfmod.PFError):
        g.autotune()
    phi, mu = I.make_ic("R", (8, 8, 32), seed=1)
    g.init_fields(phi, mu)
    g.set_variant("tuned")
    with pytest.raises(pfmod.PFError):
        g.autotune()
    g.set_variant("jit")
    rep = g.autotune(mask=pfmod.PF_MU, passes=1, reps=2)
    assert "mu" in rep and "phi" not in rep


@pytest.mark.parametrize("knobs", [dict(R1, mu_cly=2), dict(R1, mu_cly=4), R1,
                                   {"mu_rpt": 2, "mu_ty": 6, "mu_minb": 3},
                                   # taller two-rows tiles, one CTA per SM (ragged in y)
                                   {"mu_rpt": 2, "mu_ty": 16, "mu_minb": 1},
                                   {"mu_rpt": 2, "mu_ty": 10, "mu_minb": 1}])
def test_mu_sweep_layouts_bitwise(pfmod, omod, monkeypatch, knobs):
    """mu_cly > 1 (tiles of a thread-block cluster take the sides of their
    shared y edges from each other's shared memory) and mu_rpt = 2 (two tile
    rows per thread): bitwise equal to the default mu-sweep on a DS block
    with window shifts (ragged last tile in y), on a periodic block through
    the interior / shell launches of the forced exchange (cluster kernels
    fall back to the plain ones there), and <= 1e-12 from the oracle after
    one step."""
    P = I.params_c4("ds", window_check=2, window_frac=0.3)
    shape = (40, 30, 45)
    phi, mu = I.ic_lamellar(shape, seed=5, z_front=14)
    o = omod.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    o.step(1)
    op, om = o.download()
    gp, gm = gpu_run(pfmod, shape, P, phi, mu, 1, knobs, I.BC_DS)
    assert rel_linf(gp, op) <= TOL_1 and rel_linf(gm, om) <= TOL_1
    ref = gpu_run(pfmod, shape, P, phi, mu, 12, None, I.BC_DS)
    got = gpu_run(pfmod, shape, P, phi, mu, 12, knobs, I.BC_DS)
    assert np.array_equal(ref[0], got[0]) and np.array_equal(ref[1], got[1])
    Ps = I.params_stress()
    shape = (70, 32, 100)
    phi, mu = I.ic_voronoi(shape, seed=8)
    outs = []
    for force, t in (("0", None), ("0", knobs), ("1", knobs)):
        monkeypatch.setenv("PF_FORCE_EXCHANGE", force)
        outs.append(gpu_run(pfmod, shape, Ps, phi, mu, 4, t))
    for o2 in outs[1:]:
        assert np.array_equal(outs[0][0], o2[0]) and np.array_equal(outs[0][1], o2[1])


# Step schedules (tuning sched / slab; S§7 step 6 (ii), NEXT-2): the z-slab
# pipeline launches the same kernels on slabs of planes (phi shifted up one
# plane, x / y ghosts per slab, z ghosts at the ends), so it must give the
# same bits as the two full sweeps -- DS boundaries (non-periodic z), window
# shifts, ragged z extents, mu z-chunks that do not divide nz.
@pytest.mark.parametrize("slab,mu_zc,shape", [(1, 5, (23, 14, 40)), (2, 4, (37, 9, 33)), (4, 6, (30, 16, 64)),
                                              (16, 22, (21, 8, 32))])
def test_slab_schedule_bitwise(pfmod, omod, slab, mu_zc, shape):
    P = I.params_stress(window_check=4, window_frac=0.5)
    phi, mu = I.ic_lamellar(shape, seed=7, z_front=shape[0] // 2 + 2, mu_inf=tuple(P["mu_inf"]))
    outs = []
    # sched 2: the same slabs with the mu slabs on their own stream, concurrent
    # with the next phi slab (CUDA-graph steps forced on for one of them)
    for t in ({"sched": 0, "mu_zc": mu_zc}, {"sched": 1, "slab": slab, "mu_zc": mu_zc},
              {"sched": 2, "slab": slab, "mu_zc": mu_zc}, {"sched": 2, "slab": slab, "mu_zc": mu_zc, "graph": 1}):
        t = dict(t)
        graph = t.pop("graph", 0)
        if graph:
            os.environ["PF_GRAPH"] = "1"
        try:
            g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
        finally:
            os.environ.pop("PF_GRAPH", None)
        g.set_tuning(t)
        g.init_fields(phi, mu)
        g.step(9)
        outs.append((g.download(), g.state()))
        g.close()
    (p0, m0), s0 = outs[0]
    for (p1, m1), s1 in outs[1:]:
        assert s0 == s1 and s0["z_off"] > 0
        assert np.array_equal(p0, p1) and np.array_equal(m0, m1)
    o = omod.Oracle(shape, P, I.BC_DS)
    o.init(phi, mu)
    o.step(9)
    op, om = o.download()
    assert np.abs(p1 - op).max() / np.abs(op).max() <= 1e-11 and np.abs(m1 - om).max() / np.abs(om).max() <= 1e-11


def test_autotune_step_schedule(pfmod):
    """pf_autotune times the step schedules as dry steps (state untouched) and
    reports the choice."""
    shape = (48, 32, 64)
    P = I.params_c4("ds", window_check=0)
    phi, mu = I.ic_lamellar(shape, seed=3)
    g = pfmod.PhaseField(shape, P, bc=I.BC_DS)
    g.init_fields(phi, mu)
    before = g.download()
    rep = g.autotune(passes=1, reps=3, variants=True)
    after = g.download()
    assert np.array_equal(before[0], after[0]) and np.array_equal(before[1], after[1])
    assert "step" in rep and rep["step"]["sched"] in (0, 1)
    v = rep["variants"]
    assert v["chosen"] == 2 and v["fused_jit_ms"] < v["full_ms"] and v["fused_jit_ms"] < v["split_ms"], v
    assert any(c["kernel"] == "step" for c in rep["tried"])
