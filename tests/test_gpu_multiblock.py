"""Multi-block runs of the library on ONE GPU (VERDICT r1 "next" 6; SURVEY
§8(e), T4 / C.7: "the gathered global field must be bitwise equal to the
1-GPU result").

The `world` blocks of a px x py x pz decomposition are separate pf_ctx
contexts in this process, each on its own CUDA stream and stepped from its
own host thread, connected by the in-process transport of pf_api.cu
(pf_config.nccl_uid = "PFLOCAL:<name>").  Everything but the transport is the
multi-GPU code path: pack / unpack kernels, the ordered x -> y -> z stages,
the zero-copy z planes, the interior / shell overlap of the mu-sweep
(TileSel launches on the comm stream's schedule), the max-reductions of the
window trigger and the monitors.  The gathered fields must be bitwise equal
to a single-block run of the same global domain.  -m gpu.
"""
import concurrent.futures as cf
import itertools
import uuid

import numpy as np
import pytest

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pfmod():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("GPU test without a CUDA device")
    from paper_conf_sc_0003hehshhkwnr19_b200 import build, pf
    build.build()
    return pf


def run_single(pf, shape, P, bc, phi, mu, steps, variant):
    g = pf.PhaseField(shape, P, bc=bc)
    g.set_variant(variant)
    g.init_fields(phi, mu)
    g.step(steps)
    out = g.download()
    st = g.state()
    g.close()
    return out, st


def run_blocks(pf, shape, P, bc, phi, mu, steps, procs, variant, chunks=1):
    """The same run as `world` blocks stepped concurrently; returns the
    gathered global fields, the per-rank states and the monitors."""
    import torch
    world = procs[0] * procs[1] * procs[2]
    name = uuid.uuid4().hex[:16]
    blocks = []
    for r in range(world):
        s = torch.cuda.Stream()
        g = pf.PhaseField(shape, P, bc=bc, procs=procs, rank=r, world=world, stream=s, local_group=name)
        g.set_variant(variant)
        blocks.append(g)

    def work(r):
        g = blocks[r]
        (oz, oy, ox), (nz, ny, nx) = g.offset, g.local
        g.init_fields(np.ascontiguousarray(phi[:, oz:oz + nz, oy:oy + ny, ox:ox + nx]),
                      np.ascontiguousarray(mu[:, oz:oz + nz, oy:oy + ny, ox:ox + nx]))
        for _ in range(chunks):
            g.step(steps // chunks)
        mon = g.monitor()  # collective (max over ranks)
        return g.download(), g.state(), mon

    with cf.ThreadPoolExecutor(world) as ex:
        res = list(ex.map(work, range(world)))
    gp = np.empty_like(phi)
    gm = np.empty_like(mu)
    for g, ((p, m), _, _) in zip(blocks, res):
        (oz, oy, ox), (nz, ny, nx) = g.offset, g.local
        gp[:, oz:oz + nz, oy:oy + ny, ox:ox + nx] = p
        gm[:, oz:oz + nz, oy:oy + ny, ox:ox + nx] = m
    for g in blocks:
        g.close()
    return (gp, gm), [r[1] for r in res], [r[2] for r in res]


CASES = {
    # name: (global (nz, ny, nx), procs (px, py, pz), parameter set, BCs, IC)
    "x2_periodic": ((12, 16, 192), (2, 1, 1), "c4", "periodic", "V"),   # 3 mu tiles per block in x: interior + shell
    "xy2x2_stress": ((10, 40, 70), (2, 2, 1), "stress", "periodic", "R"),
    "z2_periodic": ((40, 20, 36), (1, 1, 2), "c4", "periodic", "V"),    # zero-copy z planes
    "xyz_2x2x2": ((30, 26, 66), (2, 2, 2), "c4", "periodic", "V"),
    "x3_ragged": ((9, 11, 100), (3, 1, 1), "stress", "periodic", "R"),  # uneven block extents
}


def _setup(case):
    shape, procs, pset, bcname, ic = CASES[case]
    P = I.params_c4() if pset == "c4" else I.params_stress()
    if procs[2] > 1:
        P = dict(P, G=0.0, v=0.0)  # T(k) = T0 exactly: the z split cannot change its rounding
    bc = I.BC_PERIODIC if bcname == "periodic" else I.BC_DS
    phi, mu = I.make_ic(ic, shape, seed=31)
    return shape, procs, P, bc, phi, mu


@pytest.mark.parametrize("variant", ["jit", "tuned"])
@pytest.mark.parametrize("case", sorted(CASES))
def test_blocks_bitwise_equal_single(pfmod, case, variant):
    shape, procs, P, bc, phi, mu = _setup(case)
    steps = 12
    (sp, sm), _ = run_single(pfmod, shape, P, bc, phi, mu, steps, variant)
    (bp, bm), states, mons = run_blocks(pfmod, shape, P, bc, phi, mu, steps, procs, variant, chunks=2)
    assert np.array_equal(bp, sp) and np.array_equal(bm, sm), (
        np.abs(bp - sp).max(), np.abs(bm - sm).max())
    assert all(s == states[0] for s in states)
    assert all(m == mons[0] for m in mons)  # the monitors are reduced over ranks


@pytest.mark.parametrize("env", [{}, {"PF_OVERLAP": "0"}, {"PF_ZC_EXCHANGE": "0"}, {"PF_LAYOUT": "il"}])
def test_schedules_bitwise(pfmod, monkeypatch, env):
    """Overlap on / off (the Table-2 analog), packed vs
    zero-copy z exchange and the plane-interleaved field layout give the same
    bits as one block."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    shape, procs, P, bc, phi, mu = _setup("xyz_2x2x2")
    (sp, sm), _ = run_single(pfmod, shape, P, bc, phi, mu, 8, "jit")
    (bp, bm), _, _ = run_blocks(pfmod, shape, P, bc, phi, mu, 8, procs, "jit")
    assert np.array_equal(bp, sp) and np.array_equal(bm, sm)


@pytest.mark.parametrize("procs", [(2, 2, 1), (2, 1, 1)])
def test_ds_window_blocks_bitwise(pfmod, procs):
    """Directional solidification, growth axis unsplit, blocks tiling x-y:
    the front height is max-reduced over ranks, every rank shifts the same
    planes, and the run equals one block bitwise (window shifts included)."""
    P = I.params_stress(window_check=5, window_frac=0.5)
    shape = (32, 12, 40)
    phi, mu = I.ic_lamellar(shape, seed=20191117, z_front=20, mu_inf=tuple(P["mu_inf"]))
    (sp, sm), st1 = run_single(pfmod, shape, P, I.BC_DS, phi, mu, 40, "jit")
    (bp, bm), states, _ = run_blocks(pfmod, shape, P, I.BC_DS, phi, mu, 40, procs, "jit", chunks=4)
    assert st1["z_off"] > 0
    assert all(s == st1 for s in states)
    assert np.array_equal(bp, sp) and np.array_equal(bm, sm)


@pytest.mark.parametrize("case", ["x2_periodic", "xyz_2x2x2", "ds_xy2x2"])
def test_p2_blocks_bitwise(pfmod, case):
    """The P2 parameterisation (pf_p2.cu, 3 phases / 1 mu, anisotropic phi)
    over the same transport: blocks equal one block bitwise (periodic x,
    x-y-z split, and DS with window shifts)."""
    if case == "ds_xy2x2":
        P = I.params_p2_stress(window_check=5, window_frac=0.5, v=0.05)
        shape, procs, bc = (32, 12, 40), (2, 2, 1), I.BC_DS
    else:
        P = dict(I.params_p2_stress(), G=0.0, v=0.0)
        shape, procs, _, _, _ = CASES[case]
        bc = I.BC_PERIODIC
    phi, mu = I.ic_voronoi(shape, seed=13, N=3, M=1)
    (sp, sm), st1 = run_single(pfmod, shape, P, bc, phi, mu, 20, "jit")
    (bp, bm), states, _ = run_blocks(pfmod, shape, P, bc, phi, mu, 20, procs, "jit", chunks=2)
    assert all(s == st1 for s in states)
    if case == "ds_xy2x2":
        assert st1["z_off"] > 0
    assert np.array_equal(bp, sp) and np.array_equal(bm, sm), (np.abs(bp - sp).max(), np.abs(bm - sm).max())
