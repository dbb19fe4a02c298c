"""A few P2 steps at n^3 (default 256) for ncu captures of the P2 kernels:
    ncu -k regex:k_mu_side ... python tools/p2_run.py [n] [steps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 4
g = pf.PhaseField((n, n, n), I.params_p2())
phi, mu = I.ic_voronoi((n, n, n), seed=20191117, N=3, M=1)
g.init_fields(phi, mu)
g.step(steps)
g.download()
print("p2 run ok", g.state())
