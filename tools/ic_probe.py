"""One initial condition at 256^3 for ncu: init, 12 steps (C.4 'ds', DS
boundaries, window off).  Used by tools/gpu_ic_ncu.sh to compare the sweeps'
hardware counters between IC-R and IC-L (S§8(d) D.8).
usage: python tools/ic_probe.py R|V|L"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

n = 256
P = I.params_c4("ds", window_check=0)
P["T0"] = I.ds_T0(n // 4, P["G"])
phi, mu = I.make_ic(sys.argv[1], (n, n, n), seed=20191117)
g = pf.PhaseField((n, n, n), P, bc=I.BC_DS)
g.init_fields(phi, mu)
del phi, mu
g.step(12)
torch.cuda.synchronize()
g.close()
