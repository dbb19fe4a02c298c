"""Shared helpers for the oracle pins (test infrastructure)."""
import numpy as np

BC_X_NEUMANN = {"lo": ("neumann", "periodic", "periodic"), "hi": ("neumann", "periodic", "periodic")}
BC_PERIODIC = {"lo": ("periodic",) * 3, "hi": ("periodic",) * 3}


def simple_params(N=2, M=1, eps=3.0, dx=1.0, dt=0.01, g3=10.0, dpsi=0.0, tau=1.0, liquid=None):
    """Reduced parameter set: gamma = 1, chi = I, D = 0, psi_0 = -dpsi, others 0."""
    P = dict(N=N, M=M, liquid=N - 1 if liquid is None else liquid, dx=dx, dt=dt, eps=eps,
             gamma=np.ones((N, N)) - np.eye(N), gamma3=np.zeros((N, N, N)),
             tau=np.full((N, N), tau), A0=np.array([-0.5 * np.eye(M)] * N), A1=np.zeros((N, M, M)),
             B0=np.zeros((N, M)), B1=np.zeros((N, M)), C0=np.zeros(N), C1=np.zeros(N),
             D=np.zeros((N, M, M)), T0=1.0, G=0.0, v=0.0, mu_inf=np.zeros(M))
    for a in range(N):
        for b in range(N):
            for d in range(N):
                if len({a, b, d}) == 3:
                    P["gamma3"][a, b, d] = g3
    P["C0"][0] = -dpsi
    return P


def sine_profile(u, eps):
    """Stationary two-phase profile of the obstacle model:
    phi = 1/2 + 1/2 sin(k u), k = 4/(pi eps), on |u| <= pi/(2k); 0 / 1 outside."""
    k = 4.0 / (np.pi * eps)
    w = np.pi / (2.0 * k)
    return np.where(u < -w, 0.0, np.where(u > w, 1.0, 0.5 + 0.5 * np.sin(k * np.clip(u, -w, w))))


def front_position(row, dx, start=0):
    """x where `row` (increasing through 1/2) crosses 1/2, linear interpolation."""
    i = np.nonzero((row[start:-1] < 0.5) & (row[start + 1:] >= 0.5))[0][0] + start
    return (i + 0.5 + (0.5 - row[i]) / (row[i + 1] - row[i])) * dx
