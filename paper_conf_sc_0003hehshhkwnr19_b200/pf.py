"""Thin ctypes binding of the C ABI in include/pf.h (argument marshalling only).

Every step of the method runs in the CUDA kernels of libpf.so; PyTorch only
provides device memory (the caller-owned buffers of pf_config), the stream
and, for world > 1, the process group used to broadcast the NCCL id.  There
is no CPU fallback: if libpf.so or a CUDA device is missing, this module
raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libpf.so")

PF_OK, PF_EINVAL, PF_ENOMEM, PF_ECUDA, PF_ENCCL, PF_ESTATE, PF_ENUMERIC = 0, -1, -2, -3, -4, -5, -6
GUARD_BYTE = 0xA5  # fill of the test-only guard zones (PF_TEST_GUARD_BYTES)
BC = {"periodic": 0, "neumann": 1, "dirichlet_mu": 2}
PF_HOST, PF_DEVICE = 0, 1
PF_PHI, PF_MU = 1, 2
VARIANT = {"tuned": 0, "naive": 1, "jit": 2, "split": 3}
N, M = 4, 2


class PFConfig(C.Structure):
    _fields_ = [("n_phases", C.c_int), ("n_mu", C.c_int), ("liquid", C.c_int),
                ("global_", C.c_int * 3), ("procs", C.c_int * 3),
                ("bc_lo", C.c_int * 3), ("bc_hi", C.c_int * 3),
                ("rank", C.c_int), ("world", C.c_int),
                ("nccl_uid", C.c_ubyte * 128), ("device", C.c_int), ("stream", C.c_void_p),
                ("phi", C.c_void_p * 2), ("mu", C.c_void_p * 2), ("workspace", C.c_void_p)]


class PFLayout(C.Structure):
    _fields_ = [("local", C.c_int * 3), ("offset", C.c_int * 3),
                ("pitch", C.c_int64), ("plane", C.c_int64), ("field", C.c_int64), ("x_off", C.c_int64),
                ("phi_bytes", C.c_size_t), ("mu_bytes", C.c_size_t), ("workspace_bytes", C.c_size_t)]


class PFParams(C.Structure):
    _fields_ = [("dx", C.c_double), ("dt", C.c_double), ("eps", C.c_double),
                ("gamma", C.c_double * N * N), ("gamma3", C.c_double * N * N * N), ("tau", C.c_double * N * N),
                ("A0", C.c_double * M * M * N), ("A1", C.c_double * M * M * N),
                ("B0", C.c_double * M * N), ("B1", C.c_double * M * N),
                ("C0", C.c_double * N), ("C1", C.c_double * N),
                ("D", C.c_double * M * M * N),
                ("T0", C.c_double), ("G", C.c_double), ("v", C.c_double),
                ("mu_inf", C.c_double * M), ("window_frac", C.c_double), ("window_check", C.c_int),
                ("xi_amp", C.c_double), ("xi_seed", C.c_uint32),
                ("aniso", C.c_int), ("aniso_delta", C.c_double * N * N),
                ("aniso_R", C.c_double * 3 * 3 * N * N)]


TUNING_KNOBS = ("phi_ty", "phi_minb", "phi_zc", "phi_faces6", "phi_unroll", "phi_prefetch", "phi_pfd", "phi_xsh", "phi_zrec", "phi_xghost",
                "mu_ty", "mu_tx", "mu_minb", "mu_zc", "mu_prefetch", "mu_pfd", "mu_rpf", "mu_halo_l1", "mu_fxreg",
                "mu_qreg", "mu_ldhint", "mu_hpipe", "mu_cly", "mu_rot", "mu_rpt", "phi_rpt", "mu_pers", "phi_pers", "sched", "slab", "mu_tmem",
               "mu_hcar", "mu_xshfl", "p2_phi", "p2_mu", "p2_phi_ty", "p2_phi_minb", "p2_mu_ty", "p2_mu_minb",
               "p2_phi_pd", "p2_mu_pd", "mu_atskip", "mu_hasync", "p2_mu_hasync")


class PFTuning(C.Structure):
    _fields_ = [(k, C.c_int) for k in TUNING_KNOBS]


class PFState(C.Structure):
    _fields_ = [("step", C.c_int64), ("z_off", C.c_int64)]


# every symbol include/pf.h declares (checked by tests/test_abi.py)
ABI_SYMBOLS = ["pf_query_layout", "pf_query_neighbors", "pf_create", "pf_destroy", "pf_set_params", "pf_init_fields", "pf_step",
               "pf_step_phi_only", "pf_halo_exchange", "pf_shift_window", "pf_front_height", "pf_monitor",
               "pf_set_monitors", "pf_download", "pf_get_state", "pf_set_state", "pf_set_variant", "pf_tuning_default", "pf_set_tuning",
               "pf_get_tuning", "pf_tuning_check", "pf_autotune", "pf_profile", "pf_profile_read",
               "pf_nccl_unique_id", "pf_jit_compile_only", "pf_jit_compile_only_p2", "pf_last_error", "pf_version"]

_lib = None


def load_library(path: str = LIB_PATH):
    """Load libpf.so (no CUDA device needed just to load it)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"CUDA extension missing: {path} (run __graft_entry__.build())")
    L = C.CDLL(path)
    vp, ip = C.c_void_p, C.c_int
    dp = C.POINTER(C.c_double)
    L.pf_query_layout.argtypes = [C.POINTER(PFConfig), C.POINTER(PFLayout)]
    L.pf_query_neighbors.argtypes = [C.POINTER(PFConfig), C.POINTER(ip), C.POINTER(ip)]
    L.pf_create.argtypes = [C.POINTER(PFConfig), C.POINTER(vp)]
    L.pf_destroy.argtypes = [vp]
    L.pf_set_params.argtypes = [vp, C.POINTER(PFParams)]
    L.pf_init_fields.argtypes = [vp, vp, vp, ip]
    L.pf_step.argtypes = [vp, C.c_int64]
    L.pf_step_phi_only.argtypes = [vp]
    L.pf_halo_exchange.argtypes = [vp, C.c_uint]
    L.pf_shift_window.argtypes = [vp, ip]
    L.pf_front_height.argtypes = [vp, C.POINTER(ip)]
    L.pf_monitor.argtypes = [vp, dp]
    L.pf_set_monitors.argtypes = [vp, ip, C.c_double]
    L.pf_download.argtypes = [vp, vp, vp, ip]
    L.pf_get_state.argtypes = [vp, C.POINTER(PFState)]
    L.pf_set_state.argtypes = [vp, C.POINTER(PFState)]
    L.pf_set_variant.argtypes = [vp, ip]
    L.pf_tuning_default.argtypes = [C.POINTER(PFTuning)]
    L.pf_set_tuning.argtypes = [vp, C.POINTER(PFTuning)]
    L.pf_get_tuning.argtypes = [vp, C.POINTER(PFTuning)]
    L.pf_tuning_check.argtypes = [C.POINTER(PFTuning), C.c_char_p, ip]
    L.pf_autotune.argtypes = [vp, C.c_uint, ip, ip, C.c_char_p, ip]
    L.pf_profile.argtypes = [vp, ip]
    L.pf_profile_read.argtypes = [vp, dp, C.POINTER(C.c_int64)]
    L.pf_nccl_unique_id.argtypes = [C.POINTER(C.c_ubyte)]
    L.pf_jit_compile_only.argtypes = [C.POINTER(PFParams), ip, ip, C.POINTER(PFTuning), C.c_char_p, C.c_char_p, ip]
    L.pf_jit_compile_only_p2.argtypes = [C.POINTER(PFParams), ip, ip, C.POINTER(PFTuning), C.c_char_p, C.c_char_p, ip]
    L.pf_last_error.argtypes = [vp]
    L.pf_last_error.restype = C.c_char_p
    L.pf_version.restype = C.c_char_p
    _lib = L
    return L


class PFError(RuntimeError):
    pass


def tuning_default() -> dict:
    """Built-in tuning of the specialised sweeps (+ PF_* environment overrides)."""
    t = PFTuning()
    load_library().pf_tuning_default(C.byref(t))
    return {k: int(getattr(t, k)) for k in TUNING_KNOBS}


def make_params(P: dict) -> PFParams:
    p = PFParams()
    n, m = int(P["N"]), int(P["M"])
    assert (n, m) in ((N, M), (3, 1)), "the CUDA path runs P1 (N = 4, M = 2) or P2 (N = 3, M = 1)"

    def put(dst, arr, shape):
        arr = np.asarray(arr, dtype=np.float64)
        assert arr.shape == shape, (arr.shape, shape)
        for ix in np.ndindex(*shape):
            o = dst
            for k in ix[:-1]:
                o = o[k]
            o[ix[-1]] = float(arr[ix])

    p.dx, p.dt, p.eps = float(P["dx"]), float(P["dt"]), float(P["eps"])
    put(p.gamma, P["gamma"], (n, n))
    put(p.gamma3, P["gamma3"], (n, n, n))
    put(p.tau, P["tau"], (n, n))
    put(p.A0, P["A0"], (n, m, m))
    put(p.A1, P["A1"], (n, m, m))
    put(p.B0, P["B0"], (n, m))
    put(p.B1, P["B1"], (n, m))
    put(p.C0, P["C0"], (n,))
    put(p.C1, P["C1"], (n,))
    put(p.D, P["D"], (n, m, m))
    p.T0, p.G, p.v = float(P["T0"]), float(P["G"]), float(P["v"])
    put(p.mu_inf, P["mu_inf"], (m,))
    p.aniso = int(P.get("aniso", 0))
    if p.aniso:
        put(p.aniso_delta, P["aniso_delta"], (n, n))
        put(p.aniso_R, P["aniso_R"], (n, n, 3, 3))
    p.window_frac = float(P.get("window_frac", 0.5))
    p.window_check = int(P.get("window_check", 0))
    p.xi_amp = float(P.get("xi_amp", 0.0))
    p.xi_seed = int(P.get("xi_seed", 0)) & 0xFFFFFFFF
    return p


def _tuning_struct(tuning: dict) -> PFTuning:
    t = dict(tuning_default(), **tuning)
    return PFTuning(*[int(t[k]) for k in TUNING_KNOBS])


def tuning_check(tuning: dict) -> str:
    """pf_tuning_check: "ok" or the reason the tuning is out of range."""
    log = C.create_string_buffer(256)
    load_library().pf_tuning_check(C.byref(_tuning_struct(tuning)), log, 256)
    return log.value.decode()


def jit_compile_only(params: dict, n: int = 64, cubin_path: str | None = None, tuning: dict | None = None) -> int:
    """Compile the run-time specialised kernels for `params`, an n^3 block and
    `tuning` (None: the default) without a GPU (NVRTC only); returns the
    total cubin size (mu-sweep cubin at cubin_path, phi-sweep at cubin_path.phi)."""
    p = make_params(params)
    log = C.create_string_buffer(8192)
    t = C.byref(_tuning_struct(tuning)) if tuning is not None else None
    r = load_library().pf_jit_compile_only(C.byref(p), int(params.get("liquid", 3)), int(n), t,
                                           (cubin_path or "").encode(), log, 8192)
    if r < 0:
        raise PFError(f"specialised compile failed: {log.value.decode()}")
    return r


def jit_compile_only_p2(params: dict, n: int = 64, cubin_path: str | None = None, tuning: dict | None = None) -> int:
    """As jit_compile_only for the P2 sweeps (3 phases, 1 mu): the specialised
    phi- and mu-sweep of the kernel choice in `tuning` (p2_* knobs)."""
    p = make_params(params)
    log = C.create_string_buffer(8192)
    t = C.byref(_tuning_struct(tuning)) if tuning is not None else None
    r = load_library().pf_jit_compile_only_p2(C.byref(p), int(params.get("liquid", 2)), int(n), t,
                                              (cubin_path or "").encode(), log, 8192)
    if r < 0:
        raise PFError(f"specialised P2 compile failed: {log.value.decode()}")
    return r


def make_config(shape, bc=None, liquid: int = 3, procs=(1, 1, 1), rank: int = 0, world: int = 1,
                n_phases: int = N, n_mu: int = M) -> PFConfig:
    """pf_config for a global (nz, ny, nx) domain (no buffers bound); P1
    (4 phases, 2 mu) or P2 (3 phases, 1 mu)."""
    nz, ny, nx = shape
    bc = bc or {"lo": ("periodic",) * 3, "hi": ("periodic",) * 3}
    cfg = PFConfig()
    cfg.n_phases, cfg.n_mu, cfg.liquid = int(n_phases), int(n_mu), int(liquid)
    for d, n in enumerate((nx, ny, nz)):
        cfg.global_[d] = n
        cfg.procs[d] = int(procs[d])
        cfg.bc_lo[d] = BC[bc["lo"][d]]
        cfg.bc_hi[d] = BC[bc["hi"][d]]
    cfg.rank, cfg.world = int(rank), int(world)
    return cfg


def query_layout(shape, procs=(1, 1, 1), rank: int = 0, world: int = 1, bc=None, n_phases: int = N,
                 n_mu: int = M) -> PFLayout:
    """Host-only block layout of `rank` (no GPU needed)."""
    lay = PFLayout()
    cfg = make_config(shape, bc, n_phases - 1, procs, rank, world, n_phases, n_mu)
    r = load_library().pf_query_layout(C.byref(cfg), C.byref(lay))
    if r != PF_OK:
        raise PFError(f"pf_query_layout failed ({r})")
    return lay


def query_neighbors(shape, procs=(1, 1, 1), rank: int = 0, world: int = 1, bc=None):
    """Host-only neighbour ranks (x, y, z) of `rank`: (lo, hi), -1 = boundary."""
    lo, hi = (C.c_int * 3)(), (C.c_int * 3)()
    r = load_library().pf_query_neighbors(C.byref(make_config(shape, bc, 3, procs, rank, world)), lo, hi)
    if r != PF_OK:
        raise PFError(f"pf_query_neighbors failed ({r})")
    return tuple(lo), tuple(hi)


def nccl_unique_id() -> bytes:
    buf = (C.c_ubyte * 128)()
    r = load_library().pf_nccl_unique_id(buf)
    if r != PF_OK:
        raise PFError(f"pf_nccl_unique_id failed ({r})")
    return bytes(buf)


class PhaseField:
    """One block of the global domain on one GPU (one rank).

    shape = global (nz, ny, nx); procs = rank grid (px, py, pz); bc = dict
    {"lo": (x, y, z), "hi": (x, y, z)} of "periodic" / "neumann" /
    "dirichlet_mu".  Buffers are torch tensors owned by this object.
    local_group = name: this block is rank `rank` of a decomposition whose
    `world` blocks live in this process (each stepped from its own thread);
    see pf.h (nccl_uid "PFLOCAL:").
    """

    def __init__(self, shape, params: dict, bc=None, liquid: int | None = None, procs=(1, 1, 1), rank: int = 0,
                 world: int = 1, device: int | None = None, nccl_uid: bytes | None = None, stream=None,
                 local_group: str | None = None):
        import torch
        if not torch.cuda.is_available():
            raise PFError("no CUDA device: the phase-field step has no CPU fallback")
        self.lib = load_library()
        self.torch = torch
        dev = torch.cuda.current_device() if device is None else int(device)
        self.device = torch.device("cuda", dev)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        nz, ny, nx = shape
        bc = bc or {"lo": ("periodic",) * 3, "hi": ("periodic",) * 3}
        cfg = PFConfig()
        liquid = int(params.get("liquid", 3)) if liquid is None else int(liquid)
        self.N, self.M = int(params.get("N", N)), int(params.get("M", M))
        cfg.n_phases, cfg.n_mu, cfg.liquid = self.N, self.M, liquid
        for d, n in enumerate((nx, ny, nz)):
            cfg.global_[d] = n
            cfg.procs[d] = int(procs[d])
            cfg.bc_lo[d] = BC[bc["lo"][d]]
            cfg.bc_hi[d] = BC[bc["hi"][d]]
        cfg.rank, cfg.world = int(rank), int(world)
        if local_group is not None:  # in-process transport (pf.h: "PFLOCAL:<name>")
            nccl_uid = b"PFLOCAL:" + local_group.encode()[:110] + b"\0"
        if nccl_uid is not None:
            for i, b in enumerate(nccl_uid[:128]):
                cfg.nccl_uid[i] = b
        cfg.device = dev
        cfg.stream = self.stream.cuda_stream
        lay = PFLayout()
        self._check(self.lib.pf_query_layout(C.byref(cfg), C.byref(lay)), "pf_query_layout", ctx=False)
        self.layout = lay
        self.local = (lay.local[2], lay.local[1], lay.local[0])
        self.offset = (lay.offset[2], lay.offset[1], lay.offset[0])
        u8 = torch.uint8
        # PF_TEST_GUARD_BYTES > 0 (tests only): every caller-owned buffer sits
        # between two guard zones of that many bytes filled with GUARD_BYTE;
        # close() raises if a kernel wrote into one (an out-of-bounds store
        # past the layout pf_query_layout gave)
        self._guard = int(os.environ.get("PF_TEST_GUARD_BYTES", "0"))
        gb = self._guard = (self._guard + 255) // 256 * 256

        def buf(n, zero=True):
            t = torch.empty(n + 2 * gb, dtype=u8, device=self.device)
            if gb:
                t.fill_(GUARD_BYTE)
            inner = t[gb:gb + n]
            if zero:
                inner.zero_()
            return t, inner
        self._raw = []
        self._phi, self._mu = [], []
        for i in range(2):
            for lst, n in ((self._phi, lay.phi_bytes), (self._mu, lay.mu_bytes)):
                t, inner = buf(n)
                self._raw.append(t)
                lst.append(inner)
            cfg.phi[i] = self._phi[i].data_ptr()
            cfg.mu[i] = self._mu[i].data_ptr()
        t, self._ws = buf(lay.workspace_bytes)
        self._raw.append(t)
        cfg.workspace = self._ws.data_ptr()
        self._cfg = cfg
        h = C.c_void_p()
        r = self.lib.pf_create(C.byref(cfg), C.byref(h))
        self._h = h
        if r != PF_OK:
            msg = self.lib.pf_last_error(h).decode() if h.value else ""
            raise PFError(f"pf_create failed ({r}): {msg}")
        self.set_params(params)

    # -- helpers ---------------------------------------------------------
    def _check(self, r, what, ctx=True):
        if r != PF_OK:
            msg = self.lib.pf_last_error(self._h).decode() if ctx else ""
            raise PFError(f"{what} failed ({r}): {msg}")

    def guards_intact(self) -> bool:
        """True unless a kernel stored into the guard zones around the
        caller-owned buffers (PF_TEST_GUARD_BYTES; always True without)."""
        gb = getattr(self, "_guard", 0)
        if not gb:
            return True
        self.torch.cuda.synchronize(self.device)
        for t in self._raw:
            if not (bool((t[:gb] == GUARD_BYTE).all()) and bool((t[-gb:] == GUARD_BYTE).all())):
                return False
        return True

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self.lib.pf_destroy(self._h)
            self._h = C.c_void_p()
            if not self.guards_intact():
                raise PFError("a kernel wrote outside the caller-owned buffers (guard zone changed)")

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- the ABI ---------------------------------------------------------
    def set_params(self, params: dict):
        self.params = dict(params)
        self._p = make_params(params)
        self._check(self.lib.pf_set_params(self._h, C.byref(self._p)), "pf_set_params")

    def init_fields(self, phi, mu):
        """phi [4][nz][ny][nx], mu [2][nz][ny][nx] block-local; numpy (host)
        or torch (host or cuda) float64, C-contiguous."""
        torch = self.torch
        if isinstance(phi, torch.Tensor):
            assert phi.dtype == torch.float64 and mu.dtype == torch.float64
            phi, mu = phi.contiguous(), mu.contiguous()
            where = PF_DEVICE if phi.is_cuda else PF_HOST
            pp, mp = phi.data_ptr(), mu.data_ptr()
            keep = (phi, mu)
        else:
            phi = np.ascontiguousarray(phi, dtype=np.float64)
            mu = np.ascontiguousarray(mu, dtype=np.float64)
            where = PF_HOST
            pp, mp = phi.ctypes.data, mu.ctypes.data
            keep = (phi, mu)
        assert tuple(phi.shape) == (self.N,) + self.local and tuple(mu.shape) == (self.M,) + self.local, (
            phi.shape, self.local)
        self._check(self.lib.pf_init_fields(self._h, C.c_void_p(pp), C.c_void_p(mp), where), "pf_init_fields")
        del keep

    def step(self, n: int = 1):
        self._check(self.lib.pf_step(self._h, int(n)), "pf_step")

    def step_phi_only(self):
        self._check(self.lib.pf_step_phi_only(self._h), "pf_step_phi_only")

    def halo_exchange(self, mask: int = PF_PHI | PF_MU):
        self._check(self.lib.pf_halo_exchange(self._h, int(mask)), "pf_halo_exchange")

    def shift_window(self, k: int):
        self._check(self.lib.pf_shift_window(self._h, int(k)), "pf_shift_window")

    def front_height(self) -> int:
        h = C.c_int(0)
        self._check(self.lib.pf_front_height(self._h, C.byref(h)), "pf_front_height")
        return h.value

    def monitor(self):
        out = (C.c_double * 2)()
        self._check(self.lib.pf_monitor(self._h, out), "pf_monitor")
        return float(out[0]), float(out[1])

    def set_monitors(self, every: int, tol: float = 1e-12):
        """pf_set_monitors: pf_step checks the invariants every `every` steps
        and raises PFError (PF_ENUMERIC) when they trip; 0 = off."""
        self._check(self.lib.pf_set_monitors(self._h, int(every), float(tol)), "pf_set_monitors")

    def download(self, out=None, device: bool = False):
        """Interior fields; numpy by default, torch cuda tensors if device=True,
        or into given pinned/cuda torch tensors `out=(phi, mu)`."""
        torch = self.torch
        if out is not None:
            phi, mu = out
            where = PF_DEVICE if phi.is_cuda else PF_HOST
            self._check(self.lib.pf_download(self._h, C.c_void_p(phi.data_ptr()), C.c_void_p(mu.data_ptr()), where),
                        "pf_download")
            return phi, mu
        if device:
            phi = torch.empty((self.N,) + self.local, dtype=torch.float64, device=self.device)
            mu = torch.empty((self.M,) + self.local, dtype=torch.float64, device=self.device)
            self._check(self.lib.pf_download(self._h, C.c_void_p(phi.data_ptr()), C.c_void_p(mu.data_ptr()),
                                             PF_DEVICE), "pf_download")
            return phi, mu
        phi = np.empty((self.N,) + self.local)
        mu = np.empty((self.M,) + self.local)
        self._check(self.lib.pf_download(self._h, C.c_void_p(phi.ctypes.data), C.c_void_p(mu.ctypes.data), PF_HOST),
                    "pf_download")
        return phi, mu

    def state(self):
        s = PFState()
        self._check(self.lib.pf_get_state(self._h, C.byref(s)), "pf_get_state")
        return {"step": s.step, "z_off": s.z_off}

    def set_state(self, step: int, z_off: int):
        s = PFState(int(step), int(z_off))
        self._check(self.lib.pf_set_state(self._h, C.byref(s)), "pf_set_state")

    def set_variant(self, name: str):
        self._check(self.lib.pf_set_variant(self._h, VARIANT[name]), "pf_set_variant")

    def tuning(self) -> dict:
        t = PFTuning()
        self._check(self.lib.pf_get_tuning(self._h, C.byref(t)), "pf_get_tuning")
        return {k: int(getattr(t, k)) for k in TUNING_KNOBS}

    def set_tuning(self, tuning: dict):
        """Set knobs of the specialised sweeps; unspecified knobs keep their value."""
        cur = self.tuning()
        unknown = set(tuning) - set(TUNING_KNOBS)
        if unknown:
            raise KeyError(f"unknown tuning knobs {sorted(unknown)}")
        cur.update({k: int(v) for k, v in tuning.items()})
        t = PFTuning(*[cur[k] for k in TUNING_KNOBS])
        self._check(self.lib.pf_set_tuning(self._h, C.byref(t)), "pf_set_tuning")

    def autotune(self, mask: int = PF_PHI | PF_MU, passes: int = 1, reps: int = 7, variants: bool = False) -> dict:
        """pf_autotune: coordinate search over the tuning knobs, timed on this
        block; returns the JSON report (start, best, per-kernel times, every
        candidate).  The context keeps the best tuning."""
        import json
        buf = C.create_string_buffer(1 << 16)
        if variants:  # PF_AUTOTUNE_VARIANTS: also time the full and split variants (S§8(f) NEXT-2)
            mask |= 4
        self._check(self.lib.pf_autotune(self._h, int(mask), int(passes), int(reps), buf, len(buf)), "pf_autotune")
        return json.loads(buf.value.decode())

    def profile(self, enable: bool = True):
        self._check(self.lib.pf_profile(self._h, int(enable)), "pf_profile")

    def profile_read(self):
        ms = (C.c_double * 4)()
        n = (C.c_int64 * 4)()
        self._check(self.lib.pf_profile_read(self._h, ms, n), "pf_profile_read")
        keys = ("phi_sweep", "mu_sweep", "ghost", "window")
        return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(keys)}
