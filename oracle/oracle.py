"""ctypes binding of the CPU ORACLE (oracle/pf_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__ (build + smoke)
and bench.py's cpu_baseline / ``--impl reference`` leg.  The product path
(paper_conf_sc_0003hehshhkwnr19_b200) never imports this module.

Argument marshalling only: every step of the method lives in pf_oracle.c.
Parameters come as the plain dict produced by
``paper_conf_sc_0003hehshhkwnr19_b200.inputs`` (a data-only module).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# PF_ORACLE_SRC / PF_ORACLE_LIB: an alternate (mutated) copy of the oracle
# source and where to build it -- used only by the mutation check
# (tools/oracle_mutations.py, tests/test_oracle_mutations.py).
SRC = os.environ.get("PF_ORACLE_SRC") or os.path.join(HERE, "pf_oracle.c")
HDR = os.path.join(HERE, "pf_oracle.h")
LIB = os.environ.get("PF_ORACLE_LIB") or os.path.join(HERE, "libpf_oracle.so")

MAXN, MAXM = 4, 2
BC = {"periodic": 0, "neumann": 1, "dirichlet_mu": 2}


class OrParams(C.Structure):
    _fields_ = [
        ("N", C.c_int), ("M", C.c_int), ("liquid", C.c_int),
        ("dx", C.c_double), ("dt", C.c_double), ("eps", C.c_double),
        ("gamma", C.c_double * MAXN * MAXN),
        ("gamma3", C.c_double * MAXN * MAXN * MAXN),
        ("tau", C.c_double * MAXN * MAXN),
        ("A0", C.c_double * MAXM * MAXM * MAXN),
        ("A1", C.c_double * MAXM * MAXM * MAXN),
        ("B0", C.c_double * MAXM * MAXN),
        ("B1", C.c_double * MAXM * MAXN),
        ("C0", C.c_double * MAXN), ("C1", C.c_double * MAXN),
        ("D", C.c_double * MAXM * MAXM * MAXN),
        ("T0", C.c_double), ("G", C.c_double), ("v", C.c_double),
        ("mu_inf", C.c_double * MAXM),
        ("window_frac", C.c_double), ("window_check", C.c_int),
        ("antitrapping", C.c_int), ("projection", C.c_int),
        ("xi_amp", C.c_double), ("xi_seed", C.c_uint),
        ("aniso", C.c_int),
        ("aniso_delta", C.c_double * MAXN * MAXN),
        ("aniso_R", C.c_double * 3 * 3 * MAXN * MAXN),
    ]


class OrGrid(C.Structure):
    _fields_ = [("nx", C.c_int), ("ny", C.c_int), ("nz", C.c_int),
                ("bc_lo", C.c_int * 3), ("bc_hi", C.c_int * 3)]


class OrState(C.Structure):
    _fields_ = [("step", C.c_int64), ("z_off", C.c_int64)]


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc: -O2 -ffp-contract=off, no fast-math."""
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= max(
            os.path.getmtime(SRC), os.path.getmtime(HDR)):
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = ["gcc", "-std=c99", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
           "-fPIC", "-shared", "-Wall", "-I", HERE, "-o", tmp, SRC, "-lm"]
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        dp = C.POINTER(C.c_double)
        L.oracle_create.restype = C.c_void_p
        L.oracle_create.argtypes = [C.POINTER(OrGrid), C.POINTER(OrParams)]
        L.oracle_destroy.argtypes = [C.c_void_p]
        L.oracle_init.argtypes = [C.c_void_p, dp, dp]
        L.oracle_step.argtypes = [C.c_void_p, C.c_int64]
        L.oracle_step_phi_only.argtypes = [C.c_void_p]
        L.oracle_shift_window.argtypes = [C.c_void_p, C.c_int]
        L.oracle_download.argtypes = [C.c_void_p, dp, dp]
        L.oracle_get_state.argtypes = [C.c_void_p, C.POINTER(OrState)]
        L.oracle_set_state.argtypes = [C.c_void_p, C.POINTER(OrState)]
        L.oracle_set_threads.argtypes = [C.c_int]
        L.oracle_phi_rhs.argtypes = [C.c_void_p, dp]
        L.oracle_project_simplex.argtypes = [C.c_int, dp, dp]
        L.oracle_front_height.argtypes = [C.c_void_p]
        u4 = C.POINTER(C.c_uint)
        L.oracle_philox4x32_10.argtypes = [u4, u4, u4]
        L.oracle_xi_uniforms.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int64, C.c_uint, dp]
        L.oracle_footprint.argtypes = [C.c_void_p, C.c_int, C.c_int, C.c_int, C.c_int, C.POINTER(C.c_int)]
        _lib = L
    return _lib


def _dp(a: np.ndarray):
    return a.ctypes.data_as(C.POINTER(C.c_double))


def make_params(P: dict) -> OrParams:
    """Fill the oracle's own POD struct from a parameter dict (inputs.py)."""
    p = OrParams()
    N, M = int(P["N"]), int(P["M"])
    p.N, p.M, p.liquid = N, M, int(P["liquid"])
    p.dx, p.dt, p.eps = float(P["dx"]), float(P["dt"]), float(P["eps"])

    def put(dst, arr, shape):
        arr = np.asarray(arr, dtype=np.float64)
        assert arr.shape == shape, (arr.shape, shape)
        for ix in np.ndindex(*shape):
            o = dst
            for k in ix[:-1]:
                o = o[k]
            o[ix[-1]] = float(arr[ix])

    put(p.gamma, P["gamma"], (N, N))
    put(p.gamma3, P["gamma3"], (N, N, N))
    put(p.tau, P["tau"], (N, N))
    put(p.A0, P["A0"], (N, M, M))
    put(p.A1, P["A1"], (N, M, M))
    put(p.B0, P["B0"], (N, M))
    put(p.B1, P["B1"], (N, M))
    put(p.C0, P["C0"], (N,))
    put(p.C1, P["C1"], (N,))
    put(p.D, P["D"], (N, M, M))
    p.T0, p.G, p.v = float(P["T0"]), float(P["G"]), float(P["v"])
    put(p.mu_inf, P["mu_inf"], (M,))
    p.window_frac = float(P.get("window_frac", 0.5))
    p.window_check = int(P.get("window_check", 0))
    p.antitrapping = int(P.get("antitrapping", 1))
    p.projection = int(P.get("projection", 1))
    p.xi_amp = float(P.get("xi_amp", 0.0))
    p.xi_seed = int(P.get("xi_seed", 0)) & 0xFFFFFFFF
    # P2 anisotropy (reading B6): aniso_delta[N][N], aniso_R[N][N][3][3]
    p.aniso = int(P.get("aniso", 0))
    if p.aniso:
        put(p.aniso_delta, P["aniso_delta"], (N, N))
        put(p.aniso_R, P["aniso_R"], (N, N, 3, 3))
    return p


def philox4x32_10(ctr, key):
    """Philox4x32-10 of the oracle (fluctuation term RNG)."""
    c = (C.c_uint * 4)(*[int(v) & 0xFFFFFFFF for v in ctr])
    k = (C.c_uint * 2)(*[int(v) & 0xFFFFFFFF for v in key])
    o = (C.c_uint * 4)()
    lib().oracle_philox4x32_10(c, k, o)
    return tuple(int(v) for v in o)


def xi_uniforms(x, y, z, step, seed) -> np.ndarray:
    """The four uniforms in (-1, 1) of cell (x, y, z) at step n (reading B4)."""
    out = np.empty(4)
    lib().oracle_xi_uniforms(int(x), int(y), int(z), int(step), int(seed) & 0xFFFFFFFF, _dp(out))
    return out


def project_simplex(x) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float64)
    out = np.empty_like(x)
    lib().oracle_project_simplex(int(x.size), _dp(x), _dp(out))
    return out


def set_threads(n: int) -> None:
    lib().oracle_set_threads(int(n))


class Oracle:
    """One global block (no decomposition) stepped on the host."""

    def __init__(self, shape, params: dict, bc=None):
        nz, ny, nx = shape  # arrays are [comp][z][y][x]
        self.shape = (nz, ny, nx)
        self.N, self.M = int(params["N"]), int(params["M"])
        g = OrGrid()
        g.nx, g.ny, g.nz = nx, ny, nz
        bc = bc or {"lo": ("periodic",) * 3, "hi": ("periodic",) * 3}
        for d in range(3):
            g.bc_lo[d] = BC[bc["lo"][d]]
            g.bc_hi[d] = BC[bc["hi"][d]]
        self._p = make_params(params)
        h = lib().oracle_create(C.byref(g), C.byref(self._p))
        if not h:
            raise ValueError("oracle_create rejected the configuration")
        self._h = C.c_void_p(h)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.oracle_destroy(h)
            self._h = None

    def init(self, phi, mu):
        phi = np.ascontiguousarray(phi, dtype=np.float64)
        mu = np.ascontiguousarray(mu, dtype=np.float64)
        assert phi.shape == (self.N,) + self.shape and mu.shape == (self.M,) + self.shape
        lib().oracle_init(self._h, _dp(phi), _dp(mu))

    def step(self, n: int = 1):
        lib().oracle_step(self._h, int(n))

    def step_phi_only(self):
        lib().oracle_step_phi_only(self._h)

    def shift_window(self, k: int):
        if lib().oracle_shift_window(self._h, int(k)) != 0:
            raise ValueError("bad shift")

    def download(self):
        phi = np.empty((self.N,) + self.shape)
        mu = np.empty((self.M,) + self.shape)
        lib().oracle_download(self._h, _dp(phi), _dp(mu))
        return phi, mu

    def state(self):
        s = OrState()
        lib().oracle_get_state(self._h, C.byref(s))
        return {"step": s.step, "z_off": s.z_off}

    def set_state(self, step: int, z_off: int):
        s = OrState(step, z_off)
        lib().oracle_set_state(self._h, C.byref(s))

    def phi_rhs(self):
        r = np.empty((self.N,) + self.shape)
        lib().oracle_phi_rhs(self._h, _dp(r))
        return r

    def front_height(self) -> int:
        return int(lib().oracle_front_height(self._h))

    def footprint(self, which: str, cell=(1, 1, 1)):
        k = ["phi-full", "phi-flux", "phi-cell", "mu-full", "mu-flux", "mu-cell"].index(which)
        st = C.c_int(0)
        x, y, z = cell
        n = lib().oracle_footprint(self._h, k, x, y, z, C.byref(st))
        return n, st.value
