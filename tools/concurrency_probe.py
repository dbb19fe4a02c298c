"""Probe: do the phi- and mu-sweeps gain from running concurrently?

Two independent 256^3 DS blocks (two contexts) are stepped (a) one after the
other on one stream and (b) concurrently on two streams (optionally with
different stream priorities), so that phi-sweep CTAs of one block can share
SMs with mu-sweep CTAs of the other.  Prints one JSON line.  Not a bench
number: an experiment for the fused-schedule design.
"""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
steps = 50
P = I.params_c4("ds")
P["T0"] = I.ds_T0(n // 4, P["G"])
shape = (n, n, n)
lo, hi = torch.cuda.Stream.priority_range() if hasattr(torch.cuda.Stream, "priority_range") else (0, -1)
res = {}
for mode in ("serial", "concurrent", "concurrent_prio"):
    if mode == "serial":
        s = torch.cuda.Stream()
        streams = [s, s]
    elif mode == "concurrent":
        streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    else:
        streams = [torch.cuda.Stream(priority=-1), torch.cuda.Stream(priority=0)]
    ctxs = []
    for i in range(2):
        g = pf.PhaseField(shape, P, bc=I.BC_DS, stream=streams[i])
        phi, mu = I.ic_lamellar(shape, seed=1 + i, z_front=n // 4)
        g.init_fields(phi, mu)
        ctxs.append(g)
    for g in ctxs:
        g.step(5)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(torch.cuda.current_stream())
    for s in set(streams):
        s.wait_event(e0)
    for k in range(steps):
        for g in ctxs:
            g.step(1)
    for s in set(streams):
        ev = torch.cuda.Event()
        ev.record(s)
        torch.cuda.current_stream().wait_event(ev)
    e1.record(torch.cuda.current_stream())
    e1.synchronize()
    ms = e0.elapsed_time(e1)
    res[mode] = {"ms": ms, "mlups": 2 * n ** 3 * steps / (ms * 1e-3) / 1e6}
    for g in ctxs:
        g.close()
    torch.cuda.synchronize()
print(json.dumps({"probe": "phi/mu concurrency", "n": n, "steps_per_block": steps, **res}))
