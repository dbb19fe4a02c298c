"""S§8(d) D.8 data-independence check: the sweeps are branch-free over cells,
so the step rate at 256^3 must not depend on the initial condition.  Times
100 steps (device events, after 10 warm-up steps) of the specialised kernels
on IC-R (Dirichlet-random phi on every cell), IC-V (Voronoi grains) and IC-L
(lamellae under liquid), same C.4 'ds' parameters and DS boundaries, window
off; prints one JSON line with MLUP/s per IC and the max/min spread."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

n, steps = 256, 100
P = I.params_c4("ds", window_check=0)
P["T0"] = I.ds_T0(n // 4, P["G"])
res = {}
for ic in ("R", "V", "L"):
    phi, mu = I.make_ic(ic, (n, n, n), seed=20191117)
    g = pf.PhaseField((n, n, n), P, bc=I.BC_DS)
    g.init_fields(phi, mu)
    del phi, mu
    g.step(10)
    g.profile(True)  # per-kernel events (direct launches)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(g.stream)
    g.step(steps)
    e1.record(g.stream)
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    pr = g.profile_read()
    res[ic] = {"mlups": n ** 3 * steps / (ms * 1e-3) / 1e6, "ms_per_step": ms / steps,
               "phi_ms": pr["phi_sweep"][0] / max(pr["phi_sweep"][1], 1),
               "mu_ms": pr["mu_sweep"][0] / max(pr["mu_sweep"][1], 1)}
    # the data-dependent anti-trapping skip (tuning mu_atskip) on the same state
    g.set_tuning({"mu_atskip": 1})
    g.step(3)
    g.profile(True)
    e0.record(g.stream)
    g.step(steps)
    e1.record(g.stream)
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    pr = g.profile_read()
    res[ic]["atskip"] = {"mlups": n ** 3 * steps / (ms * 1e-3) / 1e6,
                         "mu_ms": pr["mu_sweep"][0] / max(pr["mu_sweep"][1], 1)}
    g.close()
    torch.cuda.empty_cache()
v = [r["mlups"] for r in res.values()]
print(json.dumps({"check": "D.8 data independence, 256^3, C.4 ds parameters, DS boundaries, window off",
                  "steps": steps, **res, "spread": max(v) / min(v) - 1.0}))
