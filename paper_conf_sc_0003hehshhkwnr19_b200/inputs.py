"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module holds DATA ONLY: parameter sets (plain dicts of numbers) and
initial-condition generators (seeded random fields on the Gibbs simplex).
It contains none of the method's arithmetic -- no gradient, flux, potential,
projection or update -- so that the oracle (oracle/) and the product path
(paper_conf_sc_0003hehshhkwnr19_b200.pf) can both consume it without sharing
any code of the method (task rule 3; DESIGN.md §4 "input recipe").

The paper prints no parameter values (reading A19): the sets
below are synthetic and nondimensional, shaped like its P1 workload -- a
ternary eutectic with N = 4 phases (3 solids + liquid) and
K - 1 = 2 chemical potentials.
"""
from __future__ import annotations

import numpy as np

N_PHASES, N_MU, LIQUID = 4, 2, 3
T_E = 1.0  # eutectic temperature of the synthetic diagram

# compositions c_alpha at mu = 0 (B_alpha = -c0_alpha); solids then liquid
C0 = np.array([[0.04, 0.01], [0.62, 0.03], [0.01, 0.32], [0.18, 0.14]])
LEVER = np.array([0.34, 0.26, 0.40])  # lever-rule solid fractions of this diagram


def params_c4(kind: str = "periodic", **over) -> dict:
    """SURVEY C.4 set.  kind='periodic' (configs 1/3/4: G = v = 0, undercooled
    T0 = 0.99) or 'ds' (directional solidification: frozen gradient)."""
    N, M, L = N_PHASES, N_MU, LIQUID
    gamma = np.ones((N, N)) - np.eye(N)
    gamma3 = np.zeros((N, N, N))
    for a in range(N):
        for b in range(N):
            for d in range(N):
                if len({a, b, d}) == 3:
                    gamma3[a, b, d] = 10.0
    tau = np.full((N, N), 2.0)
    tau[L, :] = tau[:, L] = 1.0
    np.fill_diagonal(tau, 0.0)
    chi = np.array([0.5 * np.eye(M)] * 3 + [np.eye(M)])  # dc/dmu per phase
    A0 = -0.5 * chi
    A1 = np.zeros((N, M, M))
    b = np.array([0.1, 0.1])
    B0 = -C0.copy()
    B1 = np.zeros((N, M))
    B0[L] = -C0[L] + b * T_E
    B1[L] = -b
    s = np.array([1.0, 1.0, 1.0, 0.0])
    Cc0 = -s * T_E
    Cc1 = s.copy()
    D = np.array([0.01 * np.eye(M)] * 3 + [np.eye(M)])
    P = dict(N=N, M=M, liquid=L, dx=1.0, dt=0.04, eps=3.0,
             gamma=gamma, gamma3=gamma3, tau=tau, A0=A0, A1=A1, B0=B0, B1=B1,
             C0=Cc0, C1=Cc1, D=D, T0=0.99, G=0.0, v=0.0,
             mu_inf=np.zeros(M), window_frac=0.5, window_check=0,
             antitrapping=1, projection=1)
    if kind == "ds":
        P.update(G=1e-3, v=1e-3, window_check=10)
    elif kind != "periodic":
        raise ValueError(kind)
    P.update(over)
    return P


def ds_T0(z_front: int, G: float, dx: float = 1.0) -> float:
    """T0 that puts the isotherm T_E at the initial front plane (C.4)."""
    return T_E - G * z_front * dx


# Growing DS workload (SURVEY C.4 "tune v and G so the front advances
# steadily"): pulling speed and gradient measured with
# tools/ds_tune.py on a 256^3 block (profiles/r02_ds_tune.jsonl): at v = 0.1
# the front advances ~0.4 planes per 100 steps (the window shifts every
# ~260 steps); at v = 0.03 it stays within the P16 lever-rule band longer.
DS_BENCH = {"v": 0.1, "G": 0.02}
DS_LONG = {"v": 0.03, "G": 0.02}


def params_ds_growth(z_front: int, v: float, G: float, **over) -> dict:
    """C.4 set with the DS boundary conditions, pulling speed v and gradient
    G; the isotherm is placed so that the initial front is undercooled by
    v * tau_sl, the steady planar-front undercooling of App. A.3 (v = dpsi/tau
    with dpsi = T_E - T for the C.4 slopes s = 1), so the front moves from the
    first step on instead of waiting for the isotherm."""
    P = params_c4("ds", v=v, G=G, **over)
    P["T0"] = ds_T0(z_front, G) - v * P["tau"][0, LIQUID]
    return P


def params_stress(seed: int = 20191117, **over) -> dict:
    """SURVEY C.4 stress set S: every entry perturbed by a seeded +-20 %,
    non-diagonal chi_alpha and D_alpha, non-zero A1, G*v != 0, so that every
    term of the step is non-zero somewhere.  Parity only."""
    rng = np.random.default_rng(seed)
    P = params_c4("periodic")
    N, M = P["N"], P["M"]

    def pert(x, rel=0.2):
        return x * (1.0 + rel * rng.uniform(-1.0, 1.0, size=np.shape(x)))

    g = pert(P["gamma"])
    P["gamma"] = np.triu(g, 1) + np.triu(g, 1).T
    g3 = np.zeros((N, N, N))
    for a in range(N):
        for b in range(a + 1, N):
            for d in range(b + 1, N):
                v = max(5.0, 10.0 * (1.0 + 0.2 * rng.uniform(-1, 1)))
                for p in {(a, b, d), (a, d, b), (b, a, d), (b, d, a), (d, a, b), (d, b, a)}:
                    g3[p] = v
    P["gamma3"] = g3
    t = pert(P["tau"])
    P["tau"] = np.triu(t, 1) + np.triu(t, 1).T
    A0 = np.empty((N, M, M))
    for a in range(N):
        base = 0.5 if a != LIQUID else 1.0
        while True:
            R = rng.uniform(-0.3, 0.3, size=(M, M))
            chi = base * (np.eye(M) + 0.5 * (R + R.T))
            if np.all(np.linalg.eigvalsh(chi) > 0.2 * base):
                break
        A0[a] = -0.5 * chi
    P["A0"] = A0
    P["A1"] = 0.1 * A0 * rng.uniform(0.2, 1.0, size=(N, 1, 1))
    P["B0"] = pert(P["B0"])
    P["B1"] = 0.05 * rng.uniform(-1.0, 1.0, size=(N, M))
    P["C0"] = pert(P["C0"]) + 0.01 * rng.uniform(-1, 1, size=N)
    P["C1"] = pert(P["C1"]) + 0.01 * rng.uniform(-1, 1, size=N)
    D = np.empty((N, M, M))
    for a in range(N):
        base = 0.05 if a != LIQUID else 0.8
        D[a] = base * (np.eye(M) + rng.uniform(-0.2, 0.2, size=(M, M)))
    P["D"] = D
    P["G"] = 2e-3 * (1.0 + 0.2 * rng.uniform(-1, 1))
    P["v"] = 5e-3 * (1.0 + 0.2 * rng.uniform(-1, 1))
    P["T0"] = 0.98
    P["mu_inf"] = 0.01 * rng.uniform(-1, 1, size=M)
    P["dt"] = 0.03
    P.update(over)
    return P


def rot(axis: str, deg: float) -> np.ndarray:
    """Rotation matrix about a coordinate axis (data for the P2 grain orientations)."""
    c, s = np.cos(np.radians(deg)), np.sin(np.radians(deg))
    i, j = {"x": (1, 2), "y": (2, 0), "z": (0, 1)}[axis]
    R = np.eye(3)
    R[i, i], R[i, j], R[j, i], R[j, j] = c, -s, s, c
    return R


def params_p2(**over) -> dict:
    """P2 parameterisation: 3 phases (two
    solid grains of one phase with different orientations + liquid), 2
    components (one chemical potential), anisotropic gradient energy
    (reading B6: cubic A_ab(R_ab q) with strength delta on the solid-liquid
    pairs, the grains rotated against each other, as in Fig. 4 right:
    dendrites of different orientations).  Synthetic, nondimensional."""
    N, M, L = 3, 1, 2
    gamma = np.ones((N, N)) - np.eye(N)
    gamma3 = np.zeros((N, N, N))
    for a, b, d in ((0, 1, 2), (0, 2, 1), (1, 0, 2), (1, 2, 0), (2, 0, 1), (2, 1, 0)):
        gamma3[a, b, d] = 10.0
    tau = np.full((N, N), 2.0)
    tau[L, :] = tau[:, L] = 1.0
    np.fill_diagonal(tau, 0.0)
    chi = np.array([[[0.5]], [[0.5]], [[1.0]]])
    A0 = -0.5 * chi
    c0 = np.array([0.02, 0.02, 0.17])  # Al-rich solid, Cu-enriched liquid (binary Al-Cu-like)
    b = 0.1
    B0 = -c0[:, None].copy()
    B1 = np.zeros((N, M))
    B0[L, 0] = -c0[L] + b * T_E
    B1[L, 0] = -b
    s = np.array([1.0, 1.0, 0.0])
    D = np.array([[[0.01]], [[0.01]], [[1.0]]])
    delta = np.zeros((N, N))
    delta[0, L] = delta[L, 0] = delta[1, L] = delta[L, 1] = 0.05
    R = np.zeros((N, N, 3, 3))
    Rg = [np.eye(3), rot("y", 30.0) @ rot("z", 20.0)]
    for a in range(N):
        for bb in range(N):
            R[a, bb] = np.eye(3)
    for g in (0, 1):
        R[g, L] = R[L, g] = Rg[g]
    P = dict(N=N, M=M, liquid=L, dx=1.0, dt=0.03, eps=3.0, gamma=gamma, gamma3=gamma3, tau=tau,
             A0=A0, A1=np.zeros((N, M, M)), B0=B0, B1=B1, C0=-s * T_E, C1=s.copy(), D=D,
             T0=0.99, G=0.0, v=0.0, mu_inf=np.zeros(M), window_frac=0.5, window_check=0,
             antitrapping=1, projection=1, aniso=1, aniso_delta=delta, aniso_R=R)
    P.update(over)
    return P


def params_p2_ds(z_front: int, v: float = 0.05, G: float = 0.02, **over) -> dict:
    """P2 in directional solidification (NEXT-4 "dendritic DS", Fig. 4 right):
    params_p2 with a frozen gradient G pulled at v, the isotherm placed so
    that the initial front is undercooled by v tau_sl (as params_ds_growth),
    moving window; DS boundaries (BC_DS)."""
    P = params_p2(G=G, v=v, window_check=10, window_frac=0.5, **over)
    P["T0"] = ds_T0(z_front, G) - v * P["tau"][0, 2]
    return P


def params_p2_stress(seed: int = 20191118, **over) -> dict:
    """P2 stress set (parity only): every pair anisotropic with its own
    strength and a seeded random rotation, unequal gamma / tau, A1 != 0,
    G v != 0, mu_inf != 0."""
    rng = np.random.default_rng(seed)
    P = params_p2()
    N = 3

    def pert(x, rel=0.2):
        return x * (1.0 + rel * rng.uniform(-1.0, 1.0, size=np.shape(x)))

    g = pert(P["gamma"])
    P["gamma"] = np.triu(g, 1) + np.triu(g, 1).T
    t = pert(P["tau"])
    P["tau"] = np.triu(t, 1) + np.triu(t, 1).T
    d = rng.uniform(0.02, 0.08, size=(N, N))
    P["aniso_delta"] = np.triu(d, 1) + np.triu(d, 1).T
    R = np.zeros((N, N, 3, 3))
    for a in range(N):
        for b in range(a, N):
            Q, _ = np.linalg.qr(rng.normal(size=(3, 3)))
            Q *= np.sign(np.linalg.det(Q))
            R[a, b] = R[b, a] = Q
    P["aniso_R"] = R
    P["A1"] = 0.1 * P["A0"] * rng.uniform(0.2, 1.0, size=(N, 1, 1))
    P["B0"] = pert(P["B0"])
    P["B1"] = 0.05 * rng.uniform(-1.0, 1.0, size=(N, 1))
    P["C0"] = pert(P["C0"]) + 0.01 * rng.uniform(-1, 1, size=N)
    P["C1"] = pert(P["C1"]) + 0.01 * rng.uniform(-1, 1, size=N)
    P["D"] = pert(P["D"])
    P["G"] = 2e-3
    P["v"] = 5e-3
    P["T0"] = 0.98
    P["mu_inf"] = np.array([0.007])
    P["dt"] = 0.025
    P.update(over)
    return P


# ---------------------------------------------------------------------------
# Initial conditions.  Arrays are [component][z][y][x], float64.
# ---------------------------------------------------------------------------

def _blur(phi: np.ndarray, passes: int, axes=(1, 2, 3)) -> np.ndarray:
    """Periodic 3-point box average along each axis; an average of points on
    the simplex stays on the simplex (data preparation, not the method)."""
    for _ in range(passes):
        for ax in axes:
            phi = (phi + np.roll(phi, 1, axis=ax) + np.roll(phi, -1, axis=ax)) / 3.0
    return phi


def _mix_noise(phi: np.ndarray, rng, w: float) -> np.ndarray:
    """Convex mix with Dirichlet(1,...) samples in mixed (interface) cells
    only; pure bulk cells stay exactly pure and everything stays on the
    simplex."""
    N = phi.shape[0]
    mixed = phi.max(axis=0) < 1.0
    n = int(mixed.sum())
    if n:
        q = rng.dirichlet(np.ones(N), size=n).T
        phi[:, mixed] = (1.0 - w) * phi[:, mixed] + w * q
    return phi


def ic_random(shape, seed: int = 20191117, N: int = N_PHASES, M: int = N_MU, amp: float = 0.1):
    """IC-R: phi ~ Dirichlet(1,...,1) per cell, mu ~ U(-amp, amp)."""
    rng = np.random.default_rng(seed)
    nz, ny, nx = shape
    phi = rng.dirichlet(np.ones(N), size=(nz, ny, nx)).transpose(3, 0, 1, 2).copy()
    mu = rng.uniform(-amp, amp, size=(M, nz, ny, nx))
    return np.ascontiguousarray(phi), np.ascontiguousarray(mu)


def _nearest_seed(shape, seeds, periodic=True):
    nz, ny, nx = shape
    z = np.arange(nz)[:, None, None]
    y = np.arange(ny)[None, :, None]
    x = np.arange(nx)[None, None, :]
    best = np.full(shape, np.inf)
    lab = np.zeros(shape, dtype=np.int64)
    for i, (sz, sy, sx) in enumerate(seeds):
        dz, dy, dx = np.abs(z - sz), np.abs(y - sy), np.abs(x - sx)
        if periodic:
            dz, dy, dx = np.minimum(dz, nz - dz), np.minimum(dy, ny - dy), np.minimum(dx, nx - dx)
        d2 = dz * dz + dy * dy + dx * dx
        m = d2 < best
        best[m] = d2[m]
        lab[m] = i
    return lab


def ic_voronoi(shape, seed: int = 20191117, nseeds: int = 24, N: int = N_PHASES, M: int = N_MU,
               blur: int = 3, noise: float = 0.02):
    """IC-V (junction-rich): nseeds random grains of all N phases in the
    periodic box, one-hot, blurred, interface noise; mu = 0.01 U(-1,1)."""
    rng = np.random.default_rng(seed)
    nz, ny, nx = shape
    seeds = np.stack([rng.uniform(0, nz, nseeds), rng.uniform(0, ny, nseeds), rng.uniform(0, nx, nseeds)], 1)
    phase_of_seed = np.arange(nseeds) % N
    rng.shuffle(phase_of_seed)
    lab = phase_of_seed[_nearest_seed(shape, seeds)]
    phi = np.zeros((N, nz, ny, nx))
    for a in range(N):
        phi[a][lab == a] = 1.0
    phi = _blur(phi, blur)
    phi = _mix_noise(phi, rng, noise)
    mu = 0.01 * rng.uniform(-1, 1, size=(M, nz, ny, nx))
    return np.ascontiguousarray(phi), np.ascontiguousarray(mu)


def ic_lamellar(shape, seed: int = 20191117, z_front: int | None = None, ngrains: int | None = None,
                mu_inf=(0.0, 0.0), blur: int = 3, noise: float = 0.02):
    """IC-L (directional solidification): below z_front an x-y Voronoi of the
    3 solids in lever-rule proportions, extruded along z; liquid above."""
    rng = np.random.default_rng(seed)
    nz, ny, nx = shape
    N, M = N_PHASES, len(mu_inf)
    if z_front is None:
        z_front = max(1, nz // 4)
    if ngrains is None:
        ngrains = max(3, int(round(nx * ny / 400.0)))
    seeds2 = np.stack([np.zeros(ngrains), rng.uniform(0, ny, ngrains), rng.uniform(0, nx, ngrains)], 1)
    lab2 = _nearest_seed((1, ny, nx), seeds2)[0]
    solid_of = rng.choice(3, size=ngrains, p=LEVER / LEVER.sum())
    sl = solid_of[lab2]
    phi = np.zeros((N, nz, ny, nx))
    for a in range(3):
        phi[a, :z_front][:, sl == a] = 1.0
    phi[LIQUID, z_front:] = 1.0
    # blur: x, y periodic; along z only inside the domain (no wrap of liquid into solid)
    for _ in range(blur):
        for ax in (2, 3):
            phi = (phi + np.roll(phi, 1, axis=ax) + np.roll(phi, -1, axis=ax)) / 3.0
        up = np.concatenate([phi[:, :1], phi[:, :-1]], axis=1)
        dn = np.concatenate([phi[:, 1:], phi[:, -1:]], axis=1)
        phi = (up + phi + dn) / 3.0
    phi = _mix_noise(phi, rng, noise)
    mu = np.empty((M, nz, ny, nx))
    for i in range(M):
        mu[i] = mu_inf[i]
    return np.ascontiguousarray(phi), np.ascontiguousarray(mu)


def ic_p2_front(shape, seed: int = 20191117, z_front: int | None = None, ngrains: int | None = None,
                blur: int = 3, noise: float = 0.02):
    """P2 directional-solidification start: below z_front an x-y Voronoi of
    the two solid grains (phases 0, 1: the same solid, two orientations),
    extruded along z, liquid (phase 2) above; blurred, interface noise;
    mu = 0."""
    rng = np.random.default_rng(seed)
    nz, ny, nx = shape
    if z_front is None:
        z_front = max(1, nz // 4)
    if ngrains is None:
        ngrains = max(2, int(round(nx * ny / 2000.0)))
    seeds2 = np.stack([np.zeros(ngrains), rng.uniform(0, ny, ngrains), rng.uniform(0, nx, ngrains)], 1)
    lab2 = _nearest_seed((1, ny, nx), seeds2)[0] % 2
    phi = np.zeros((3, nz, ny, nx))
    for a in range(2):
        phi[a, :z_front][:, lab2 == a] = 1.0
    phi[2, z_front:] = 1.0
    for _ in range(blur):
        for ax in (2, 3):
            phi = (phi + np.roll(phi, 1, axis=ax) + np.roll(phi, -1, axis=ax)) / 3.0
        up = np.concatenate([phi[:, :1], phi[:, :-1]], axis=1)
        dn = np.concatenate([phi[:, 1:], phi[:, -1:]], axis=1)
        phi = (up + phi + dn) / 3.0
    phi = _mix_noise(phi, rng, noise)
    return np.ascontiguousarray(phi), np.zeros((1, nz, ny, nx))


def make_ic(kind: str, shape, seed: int = 20191117, **kw):
    if kind == "R":
        return ic_random(shape, seed, **kw)
    if kind == "V":
        return ic_voronoi(shape, seed, **kw)
    if kind == "L":
        return ic_lamellar(shape, seed, **kw)
    raise ValueError(kind)


BC_PERIODIC = {"lo": ("periodic",) * 3, "hi": ("periodic",) * 3}
BC_DS = {"lo": ("periodic", "periodic", "neumann"), "hi": ("periodic", "periodic", "dirichlet_mu")}
