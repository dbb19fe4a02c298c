"""JIT vs generic P2 (3 steps, 18x21x37, IC-V): max |diff| of phi and mu, for
the NVRTC options in PF_NVRTC_OPTS (build experiments on the specialisation)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

for pset in ("p2", "p2_stress"):
    P = {"p2": I.params_p2(), "p2_stress": I.params_p2_stress()}[pset]
    shape = (18, 21, 37)
    phi, mu = I.ic_voronoi(shape, seed=13, N=3, M=1)
    outs = []
    for variant in ("jit", "tuned"):
        g = pf.PhaseField(shape, P)
        g.set_variant(variant)
        g.init_fields(phi, mu)
        g.step(int(os.environ.get("STEPS", "3")))
        outs.append(g.download())
        g.close()
    dp = np.abs(outs[0][0] - outs[1][0]).max()
    dm = np.abs(outs[0][1] - outs[1][1]).max()
    nm = int((outs[0][1] != outs[1][1]).sum())
    print(os.environ.get("PF_NVRTC_OPTS", "-"), pset, "phi", dp, "mu", dm, "n_mu_diff", nm, flush=True)
