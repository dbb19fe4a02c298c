"""Small run of every kernel of the library for compute-sanitizer
(tests/test_gpu_aux.py runs it under memcheck and racecheck): a ragged DS
block with the stress parameters (mu_inf != 0, window shifts, fluctuation
term) stepped with the specialised (jit), the generic (tuned) and the naive
sweeps, plus the forced pack / unpack exchange path.

    compute-sanitizer --tool memcheck --error-exitcode 1 python tools/sanitize_run.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from paper_conf_sc_0003hehshhkwnr19_b200 import inputs as I  # noqa: E402
from paper_conf_sc_0003hehshhkwnr19_b200 import pf  # noqa: E402


def main():
    shape = (19, 13, 37)  # ragged in every direction (tiles of 32 x 8 / 32 x 4, z-chunks)
    P = I.params_stress(window_check=2, window_frac=0.5, xi_amp=0.02, xi_seed=3)
    phi, mu = I.ic_lamellar(shape, seed=5, z_front=12, mu_inf=tuple(P["mu_inf"]))
    outs = []
    for variant in sys.argv[1:] or ["jit", "tuned", "naive"]:
        g = pf.PhaseField(shape, P, bc=I.BC_DS)
        g.set_variant(variant)
        g.init_fields(phi, mu)
        g.step(4)
        g.monitor()
        g.front_height()
        outs.append(g.download())
        g.close()
    for p, m in outs[1:]:
        assert np.abs(p - outs[0][0]).max() < 1e-12 and np.abs(m - outs[0][1]).max() < 1e-12
    print("sanitize run ok", len(outs))


if __name__ == "__main__":
    main()
