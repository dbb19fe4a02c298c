"""Probe: per-step time with and without CUDA-graph step runs (PF_GRAPH).
Prints one JSON line per (shape, mode).  Not a bench number."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

for n, kind, steps in ((32, "periodic", 500), (64, "ds", 500), (256, "ds", 200)):
    for mode in ("1", "0", "1"):
        os.environ["PF_GRAPH"] = mode
        if kind == "ds":
            P = I.params_c4("ds", window_check=10, window_frac=0.5)
            P["T0"] = I.ds_T0(n // 4, P["G"])
            bc = I.BC_DS
            phi, mu = I.ic_lamellar((n, n, n), seed=1, z_front=n // 4)
        else:
            P, bc = I.params_c4(), None
            phi, mu = I.ic_voronoi((n, n, n), seed=1)
        g = pf.PhaseField((n, n, n), P, bc=bc)
        g.init_fields(phi, mu)
        g.step(20)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(g.stream)
        g.step(steps)
        e1.record(g.stream)
        e1.synchronize()
        ms = e0.elapsed_time(e1)
        out = g.download()
        print(json.dumps({"n": n, "kind": kind, "graph": mode, "us_per_step": 1e3 * ms / steps,
                          "mlups": n ** 3 * steps / (ms * 1e-3) / 1e6, "state": g.state(),
                          "checksum": float(out[1].sum())}), flush=True)
        g.close()
