"""Small run of every kernel family of the library for compute-sanitizer
(tests/test_gpu_aux.py runs it under memcheck and racecheck): a ragged DS
block with the stress parameters (mu_inf != 0, window shifts, fluctuation
term) stepped with

  * the specialised (jit), generic (tuned), naive and split sweeps,
  * specialised tunings that select other kernel bodies: persistent
    phi / mu CTAs, the TMEM-carried side of the two-rows mu-sweep, one row
    per thread, cluster kernels, and the z-slab step schedule,
  * the P2 kernels (z-marching phi, side-staged and z-marching mu,
    one-thread-per-cell),
  * a 2 x 2 x 1 multi-block run over the in-process transport (pack /
    unpack kernels, zero-copy z planes, interior / shell overlap).

    compute-sanitizer --tool memcheck --error-exitcode 1 python tools/sanitize_run.py [groups...]

groups: jit tuned naive split tunings p2 multiblock (default: all).
"""
import concurrent.futures as cf
import os
import sys
import uuid

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

SHAPE = (19, 13, 37)  # ragged in every direction (tiles of 32 x 8 / 32 x 4, z-chunks)
TUNINGS = [
    {"mu_pers": 1, "phi_pers": 1},
    {"mu_tmem": 1, "mu_zc": 7, "mu_ty": 6, "mu_minb": 3},
    {"mu_rpt": 1, "mu_ty": 4, "mu_minb": 3, "mu_cly": 2, "phi_xsh": 1},
    {"sched": 1, "slab": 2, "mu_zc": 5},
]


def p1_run(variant=None, tuning=None, steps=4):
    P = I.params_stress(window_check=2, window_frac=0.5, xi_amp=0.02, xi_seed=3)
    phi, mu = I.ic_lamellar(SHAPE, seed=5, z_front=12, mu_inf=tuple(P["mu_inf"]))
    g = pf.PhaseField(SHAPE, P, bc=I.BC_DS)
    if variant:
        g.set_variant(variant)
    if tuning:
        g.set_tuning(tuning)
    g.init_fields(phi, mu)
    g.step(steps)
    g.monitor()
    g.front_height()
    out = g.download()
    g.close()
    return out


def p2_runs():
    outs = []
    P = I.params_p2_stress(window_check=2, window_frac=0.5, v=0.05)
    phi, mu = I.ic_voronoi((20, 12, 33), seed=5, N=3, M=1)
    for naive, kmu, kphi in (("0", "side", "side"), ("0", "march", "march"), ("1", "side", "side")):
        os.environ["PF_P2_NAIVE"] = naive
        os.environ["PF_P2_MU"] = kmu
        os.environ["PF_P2_PHI"] = kphi
        g = pf.PhaseField((20, 12, 33), P, bc=I.BC_DS)
        g.init_fields(phi, mu)
        g.step(3)
        g.monitor()
        outs.append(g.download())
        g.close()
    os.environ.pop("PF_P2_NAIVE", None)
    os.environ.pop("PF_P2_MU", None)
    os.environ.pop("PF_P2_PHI", None)
    return outs


def multiblock_run(procs=(2, 2, 1), steps=4):
    import torch
    P = I.params_stress(window_check=2, window_frac=0.5, xi_amp=0.02, xi_seed=3)
    shape = (20, 12, 36)
    phi, mu = I.ic_lamellar(shape, seed=5, z_front=12, mu_inf=tuple(P["mu_inf"]))
    world = procs[0] * procs[1] * procs[2]
    name = uuid.uuid4().hex[:16]
    blocks = [pf.PhaseField(shape, P, bc=I.BC_DS, procs=procs, rank=r, world=world, stream=torch.cuda.Stream(),
                            local_group=name) for r in range(world)]

    def work(r):
        g = blocks[r]
        (oz, oy, ox), (nz, ny, nx) = g.offset, g.local
        g.init_fields(np.ascontiguousarray(phi[:, oz:oz + nz, oy:oy + ny, ox:ox + nx]),
                      np.ascontiguousarray(mu[:, oz:oz + nz, oy:oy + ny, ox:ox + nx]))
        g.step(steps)
        g.monitor()
        return g.download()

    with cf.ThreadPoolExecutor(world) as ex:
        res = list(ex.map(work, range(world)))
    gp, gm = np.empty_like(phi), np.empty_like(mu)
    for g, (p, m) in zip(blocks, res):
        (oz, oy, ox), (nz, ny, nx) = g.offset, g.local
        gp[:, oz:oz + nz, oy:oy + ny, ox:ox + nx] = p
        gm[:, oz:oz + nz, oy:oy + ny, ox:ox + nx] = m
    for g in blocks:
        g.close()
    g1 = pf.PhaseField(shape, P, bc=I.BC_DS)
    g1.init_fields(phi, mu)
    g1.step(steps)
    ref = g1.download()
    g1.close()
    assert np.array_equal(gp, ref[0]) and np.array_equal(gm, ref[1]), "multi-block run differs"


def close(a, b):
    return np.abs(a[0] - b[0]).max() < 1e-12 and np.abs(a[1] - b[1]).max() < 1e-12


def main():
    groups = sys.argv[1:] or ["jit", "tuned", "naive", "split", "tunings", "p2", "multiblock"]
    outs, n = [], 0
    for v in ("jit", "tuned", "naive", "split"):
        if v in groups:
            outs.append(p1_run(v))
    if "tunings" in groups:
        outs += [p1_run("jit", t) for t in TUNINGS]
    for o in outs[1:]:
        assert close(o, outs[0]), "variants / tunings disagree"
    n += len(outs)
    if "p2" in groups:
        a, b, c = p2_runs()
        assert close(a, b) and close(a, c), "P2 kernels disagree"
        n += 3
    if "multiblock" in groups:
        multiblock_run()
        n += 1
    print("sanitize run ok", n)


if __name__ == "__main__":
    main()
