"""Time the P2 sweeps at 256^3 (params_p2, IC-V) for explicit tunings:
    python tools/p2_ab.py '{json}' ['{json}' ...]
one JSON line per tuning: ms per step, phi / mu sweep ms (pf_profile events)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

n = 256
phi, mu = I.ic_voronoi((n, n, n), seed=20191117, N=3, M=1)
for arg in sys.argv[1:]:
    tun = json.loads(arg)
    g = pf.PhaseField((n, n, n), I.params_p2())
    g.set_tuning(tun)
    g.init_fields(phi, mu)
    g.step(5)
    g.profile(True)
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s0.record(g.stream)
    g.step(40)
    s1.record(g.stream)
    s1.synchronize()
    ms = s0.elapsed_time(s1) / 40
    pr = g.profile_read()
    print(json.dumps({"tuning": tun, "ms_per_step": ms, "mlups": n ** 3 / (ms * 1e-3) / 1e6,
                      "phi_ms": pr["phi_sweep"][0] / max(pr["phi_sweep"][1], 1),
                      "mu_ms": pr["mu_sweep"][0] / max(pr["mu_sweep"][1], 1)}), flush=True)
    g.close()
