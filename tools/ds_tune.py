"""Choose the pulling speed v and gradient G of the DS workload so that the
front advances and the moving window fires (SURVEY C.4:
"Tune v and G so the front advances steadily").

For each (v, G) the 256^2 x nz DS block starts from IC-L with the front at
z_front and the isotherm placed so that the front is undercooled by v*tau_sl
(the steady planar-front undercooling of App. A.3, v = dpsi/tau); the run
reports z_off, the front height and the P16 lamellae fractions every
`--check` steps.

    python tools/ds_tune.py [--shape 256,256,256] [--steps 4000] [--check 500]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402
from config5 import ic_lamellar_device, lamellae  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--shape", default="256,256,256", help="nz,ny,nx")
    ap.add_argument("--steps", type=int, default=4000)
    ap.add_argument("--check", type=int, default=500)
    ap.add_argument("--vs", default="0.1,0.2,0.4")
    ap.add_argument("--Gs", default="0.02,0.05")
    ap.add_argument("--zf", type=float, default=0.45, help="initial front height / nz")
    args = ap.parse_args()
    shape = tuple(int(v) for v in args.shape.split(","))
    nz = shape[0]
    dev = torch.device("cuda", 0)
    lever = [float(v) for v in I.LEVER / I.LEVER.sum()]
    for v in [float(x) for x in args.vs.split(",")]:
        for G in [float(x) for x in args.Gs.split(",")]:
            z_front = int(args.zf * nz)
            P = I.params_c4("ds", window_check=10, window_frac=0.5, v=v, G=G)
            P["T0"] = I.ds_T0(z_front, G) - v * 1.0  # undercooled by v tau_sl at the front
            g = pf.PhaseField(shape, P, bc=I.BC_DS, device=0)
            phi, mu = ic_lamellar_device(shape, 20191117, z_front, dev)
            g.init_fields(phi, mu)
            del phi, mu
            done = 0
            rows = []
            while True:
                ph, _ = g.download(device=True)
                H = g.front_height()
                fr = lamellae(ph[:, max(0, H - 20)])
                err, mn = g.monitor()
                st = g.state()
                rows.append({"step": st["step"], "z_off": st["z_off"], "H": H,
                             "fr": [round(f, 3) for f in fr], "sum_err": err, "min_phi": mn})
                del ph
                if done >= args.steps:
                    break
                g.step(args.check)
                done += args.check
            ok = all(all(abs(f - l) <= 0.1 for f, l in zip(r["fr"], lever)) for r in rows)
            shifts_per_100 = rows[-1]["z_off"] / max(args.steps, 1) * 100
            print(json.dumps({"v": v, "G": G, "z_front": z_front, "z_off_per_100_steps": shifts_per_100,
                              "lamellae_ok": ok, "rows": rows}), flush=True)
            g.close()
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
