// pf_p2.cu -- the P2 parameterisation of the paper (SURVEY §8(f) NEXT-4,
// P:L1199-1213): 3 phases, 2 components (one chemical potential), and an
// anisotropic gradient energy density a = sum_{a<b} gamma_ab A_ab(R_ab q_ab)^2
// |q_ab|^2 (eq. 4) with the cubic A of reading B6:
//   A(p) = 1 - delta (3 - 4 sum_i p_i^4 / |p|^4),  p = R q.
// The staggered phi flux d a / d(grad phi_a) then needs the whole face
// gradient (normal difference + mean of the two tangential central
// differences, eq. 11 / reading A9): a 19-point phi stencil, which is what
// makes phi the heavy kernel of P2 (Table 1: 3968 normalised FLOPs,
// P:L1234-1243).  The mu equation (eqs. 8-10) is the P1 one with M = 1.
//
// One thread per cell, every face evaluated by both of its cells (the
// paper's "full" kernels): the first B200 version of P2,
// written from the paper; parity against the oracle in tests/test_gpu_p2.py.
// Independent of oracle/ (no shared code).
#include <math.h>

#include "pf_internal.h"

namespace pf {
namespace p2 {

constexpr int N3 = 3, NS = 2;  // phases, solids

struct Params {
  double dx, dt, eps, inv_dx, dt_over_eps, at_c, dTdt, Tbase, Tdz;
  double g[N3][N3], og[N3][N3];  // gamma_ab, 16/pi^2 gamma_ab
  double g3;                     // gamma_012
  double tau[N3][N3], inv_tau_mean;
  double A0[N3], A1[N3], B0[N3], B1[N3], C0[N3], C1[N3];  // psi_a = A mu^2 + B mu + C (M = 1), affine in T
  double D[N3];
  double delta[N3][N3];
  double R[N3][N3][9];  // R_ab row-major
  int liquid, aniso;
  double mu_inf;
};

__device__ __forceinline__ double h_of(double x) { return x * x * (3.0 - 2.0 * x); }
__device__ __forceinline__ double dh_of(double x) { return 6.0 * x * (1.0 - x); }

// grad_q f, f(q) = A(R q)^2 |q|^2 (reading B6); 0 at q = 0 (f is C^1 there)
__device__ __forceinline__ void aniso_grad(const Params& P, int a, int b, const double q[3], double out[3]) {
  const double* R = P.R[a][b];
  const double delta = P.delta[a][b];
  double v[3];
#pragma unroll
  for (int i = 0; i < 3; ++i) v[i] = fma(R[3 * i], q[0], fma(R[3 * i + 1], q[1], R[3 * i + 2] * q[2]));
  const double n2 = fma(v[0], v[0], fma(v[1], v[1], v[2] * v[2]));
  if (n2 == 0.0) {
    out[0] = out[1] = out[2] = 0.0;
    return;
  }
  double s4 = 0.0;
#pragma unroll
  for (int i = 0; i < 3; ++i) s4 = fma(v[i] * v[i], v[i] * v[i], s4);
  const double i4 = 1.0 / (n2 * n2);
  const double A = 1.0 - delta * (3.0 - 4.0 * s4 * i4);
  double gp[3];
#pragma unroll
  for (int i = 0; i < 3; ++i) {
    const double dA = 16.0 * delta * (v[i] * v[i] * v[i] * i4 - s4 * v[i] * i4 / n2);
    gp[i] = 2.0 * A * fma(dA, n2, A * v[i]);
  }
#pragma unroll
  for (int j = 0; j < 3; ++j) out[j] = fma(R[j], gp[0], fma(R[3 + j], gp[1], R[6 + j] * gp[2]));
}

// staggered phi flux (d-component of d a / d grad phi_a) at the face p | p+e_d;
// f = phi_src, c = cell offset of p, st[d] = stride of axis d
__device__ __forceinline__ void phi_face(const Params& P, const double* __restrict__ f, i64 F, i64 c, int d,
                                         const i64 st[3], double j[N3]) {
  const i64 sn = st[d];
  double pb[N3], G[N3][3];
#pragma unroll
  for (int b = 0; b < N3; ++b) {
    const double vp = __ldg(f + b * F + c), vq = __ldg(f + b * F + c + sn);
    pb[b] = 0.5 * (vp + vq);
#pragma unroll
    for (int e = 0; e < 3; ++e) {
      if (e == d) {
        G[b][e] = (vq - vp) * P.inv_dx;
      } else {
        const i64 t = st[e];
        G[b][e] = ((__ldg(f + b * F + c + t) - __ldg(f + b * F + c - t)) +
                   (__ldg(f + b * F + c + sn + t) - __ldg(f + b * F + c + sn - t))) *
                  (0.25 * P.inv_dx);
      }
    }
  }
#pragma unroll
  for (int a = 0; a < N3; ++a) j[a] = 0.0;
  if (!P.aniso) {  // isotropic (A = 1): 2 sum_b gamma_ab pb_b (pb_b G_a,d - pb_a G_b,d)
#pragma unroll
    for (int a = 0; a < N3; ++a)
#pragma unroll
      for (int b = 0; b < N3; ++b)
        if (b != a) j[a] = fma(2.0 * P.g[a][b] * pb[b], fma(pb[b], G[a][d], -pb[a] * G[b][d]), j[a]);
    return;
  }
  // one grad f per pair: q_ba = -q_ab and grad f is odd
#pragma unroll
  for (int a = 0; a < N3; ++a)
#pragma unroll
    for (int b = a + 1; b < N3; ++b) {
      double q[3], gf[3];
#pragma unroll
      for (int e = 0; e < 3; ++e) q[e] = fma(pb[a], G[b][e], -pb[b] * G[a][e]);
      aniso_grad(P, a, b, q, gf);
      j[a] = fma(-P.g[a][b] * pb[b], gf[d], j[a]);
      j[b] = fma(P.g[a][b] * pb[a], gf[d], j[b]);
    }
}

__device__ __forceinline__ void project3(double x[N3]) {
  double u0 = x[0], u1 = x[1], u2 = x[2], t;
  if (u1 > u0) { t = u0; u0 = u1; u1 = t; }
  if (u2 > u1) { t = u1; u1 = u2; u2 = t; }
  if (u1 > u0) { t = u0; u0 = u1; u1 = t; }
  const double s2 = u0 + u1, s3 = s2 + u2;
  double th = u0 - 1.0;
  th = fmax(th, (s2 - 1.0) * 0.5);
  th = fmax(th, (s3 - 1.0) * (1.0 / 3.0));
#pragma unroll
  for (int a = 0; a < N3; ++a) x[a] = fmax(x[a] - th, 0.0);
}

__global__ void __launch_bounds__(256) k_phi(Params P, Geom g, const double* __restrict__ ps,
                                             const double* __restrict__ ms, double* __restrict__ pd) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const i64 c = g.at(x, y, z), F = g.field;
  const i64 st[3] = {1, g.pitch, g.plane};
  double ph[N3], gd[N3][3], div[N3] = {0.0, 0.0, 0.0};
#pragma unroll
  for (int a = 0; a < N3; ++a) ph[a] = __ldg(ps + a * F + c);
  // 1. divergence of the staggered fluxes (eq. 11)
#pragma unroll 1
  for (int d = 0; d < 3; ++d) {
    double jp[N3], jm[N3];
    phi_face(P, ps, F, c, d, st, jp);
    phi_face(P, ps, F, c - st[d], d, st, jm);
#pragma unroll
    for (int a = 0; a < N3; ++a) div[a] += (jp[a] - jm[a]) * P.inv_dx;
  }
  // 2. cell-centred gradients (central differences) [A10]
#pragma unroll
  for (int b = 0; b < N3; ++b)
#pragma unroll
    for (int d = 0; d < 3; ++d)
      gd[b][d] = (__ldg(ps + b * F + c + st[d]) - __ldg(ps + b * F + c - st[d])) * (0.5 * P.inv_dx);
  const double mu = __ldg(ms + c);
  const double T = fma(P.Tdz, (double)z, P.Tbase);
  // da/dphi_a = sum_{b != a} gamma_ab grad_q f(q_ab) . g_b,  q_ab = phi_a g_b - phi_b g_a
  double dad[N3] = {0.0, 0.0, 0.0};
#pragma unroll
  for (int a = 0; a < N3; ++a)
#pragma unroll
    for (int b = a + 1; b < N3; ++b) {
      double q[3], gf[3];
#pragma unroll
      for (int e = 0; e < 3; ++e) q[e] = fma(ph[a], gd[b][e], -ph[b] * gd[a][e]);
      if (P.aniso) {
        aniso_grad(P, a, b, q, gf);
      } else {
#pragma unroll
        for (int e = 0; e < 3; ++e) gf[e] = 2.0 * q[e];
      }
      dad[a] = fma(P.g[a][b], fma(gf[0], gd[b][0], fma(gf[1], gd[b][1], gf[2] * gd[b][2])), dad[a]);
      dad[b] = fma(-P.g[a][b], fma(gf[0], gd[a][0], fma(gf[1], gd[a][1], gf[2] * gd[a][2])), dad[b]);
    }
  double r[N3];
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    double om = 0.0;
#pragma unroll
    for (int b = 0; b < N3; ++b)
      if (b != a) om = fma(P.og[a][b], ph[b], om);
    const int b1 = a == 0 ? 1 : 0, b2 = a == 2 ? 1 : 2;  // the other two phases
    om = fma(P.g3, ph[b1] * ph[b2], om);
    const double A = fma(P.A1[a], T, P.A0[a]), B = fma(P.B1[a], T, P.B0[a]), C = fma(P.C1[a], T, P.C0[a]);
    const double psi = fma(A * mu, mu, fma(B, mu, C));
    r[a] = fma(P.eps, dad[a] - div[a], fma(om, 1.0 / P.eps, psi * dh_of(ph[a])));
  }
  // tau = sum tau_ab phi_a phi_b / sum phi_a phi_b [A5]; Euler with the Lagrange multiplier
  double num = 0.0, den = 0.0;
#pragma unroll
  for (int a = 0; a < N3; ++a)
#pragma unroll
    for (int b = a + 1; b < N3; ++b) {
      num = fma(P.tau[a][b], ph[a] * ph[b], num);
      den = fma(ph[a], ph[b], den);
    }
  const double f = den != 0.0 ? P.dt_over_eps * (den / num) : P.dt_over_eps * P.inv_tau_mean;
  const double rbar = (r[0] + r[1] + r[2]) * (1.0 / 3.0);
  double out[N3];
#pragma unroll
  for (int a = 0; a < N3; ++a) out[a] = fma(f, rbar - r[a], ph[a]);
  project3(out);
#pragma unroll
  for (int a = 0; a < N3; ++a) pd[a * F + c] = out[a];
}

// mu flux F = M grad mu - J_at at the face p | p+e_d (eqs. 8-10) [A7-A11], M = 1
__device__ __forceinline__ double mu_face(const Params& P, const double* __restrict__ ps,
                                          const double* __restrict__ pd, const double* __restrict__ ms, i64 F, i64 c,
                                          int d, const i64 st[3], double Tf) {
  const int L = P.liquid;
  const i64 sn = st[d];
  double pb[N3], G[N3][3], dtp[N3];
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    const double vp = __ldg(ps + a * F + c), vq = __ldg(ps + a * F + c + sn);
    pb[a] = 0.5 * (vp + vq);
#pragma unroll
    for (int e = 0; e < 3; ++e) {
      if (e == d) {
        G[a][e] = (vq - vp) * P.inv_dx;
      } else {
        const i64 t = st[e];
        G[a][e] = ((__ldg(ps + a * F + c + t) - __ldg(ps + a * F + c - t)) +
                   (__ldg(ps + a * F + c + sn + t) - __ldg(ps + a * F + c + sn - t))) *
                  (0.25 * P.inv_dx);
      }
    }
    dtp[a] = ((__ldg(pd + a * F + c) - vp) + (__ldg(pd + a * F + c + sn) - vq)) * (0.5 / P.dt);
  }
  const double mp = __ldg(ms + c), mq = __ldg(ms + c + sn);
  const double mb = 0.5 * (mp + mq), dmu = (mq - mp) * P.inv_dx;
  // eq. 9: M = sum_a g(pb_a) D_a chi_a(T_f), chi_a = -2 A_a, g(x) = x [A4, A7]
  double Mf = 0.0;
#pragma unroll
  for (int a = 0; a < N3; ++a) Mf = fma(pb[a] * P.D[a], -2.0 * fma(P.A1[a], Tf, P.A0[a]), Mf);
  double Fl = Mf * dmu;
  // eq. 10: J_at = (pi eps/4) sum_{s != l} g_s h_l / sqrt(phi_s phi_l) d_t phi_s (n_s . n_l)(c_l - c_s) n_s,d
  const double nl2 = fma(G[L][0], G[L][0], fma(G[L][1], G[L][1], G[L][2] * G[L][2]));
  const double cl = fma(-2.0 * fma(P.A1[L], Tf, P.A0[L]), mb, -fma(P.B1[L], Tf, P.B0[L]));
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    if (a == L) continue;
    const double na2 = fma(G[a][0], G[a][0], fma(G[a][1], G[a][1], G[a][2] * G[a][2]));
    if (!(pb[a] > 0.0 && pb[L] > 0.0 && na2 > 0.0 && nl2 > 0.0)) continue;  // [A11] exact-zero guards
    const double nra = sqrt(na2), nrl = sqrt(nl2);
    const double dot = (G[a][0] * G[L][0] + G[a][1] * G[L][1] + G[a][2] * G[L][2]) / (nra * nrl);
    const double w = P.at_c * pb[a] * h_of(pb[L]) / sqrt(pb[a] * pb[L]) * dtp[a] * dot;
    const double ca = fma(-2.0 * fma(P.A1[a], Tf, P.A0[a]), mb, -fma(P.B1[a], Tf, P.B0[a]));
    Fl -= w * (cl - ca) * (G[a][d] / nra);
  }
  return Fl;
}

__global__ void __launch_bounds__(256) k_mu(Params P, Geom g, const double* __restrict__ ps,
                                            const double* __restrict__ pd, const double* __restrict__ ms,
                                            double* __restrict__ md) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const i64 c = g.at(x, y, z), F = g.field;
  const i64 st[3] = {1, g.pitch, g.plane};
  const double T = fma(P.Tdz, (double)z, P.Tbase);
  double div = 0.0;
#pragma unroll 1
  for (int d = 0; d < 3; ++d) {
    const double Tp = d == 2 ? fma(P.Tdz, z + 0.5, P.Tbase) : T, Tm = d == 2 ? fma(P.Tdz, z - 0.5, P.Tbase) : T;
    div += (mu_face(P, ps, pd, ms, F, c, d, st, Tp) - mu_face(P, ps, pd, ms, F, c - st[d], d, st, Tm)) * P.inv_dx;
  }
  const double mu = __ldg(ms + c);
  double chi = 0.0, S = 0.0, Q = 0.0;
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    const double ph = __ldg(ps + a * F + c), phn = __ldg(pd + a * F + c);
    const double A = fma(P.A1[a], T, P.A0[a]), B = fma(P.B1[a], T, P.B0[a]);
    const double h = h_of(ph);
    chi = fma(h, -2.0 * A, chi);                                            // chi = sum h_a chi_a
    S = fma(fma(-2.0 * A, mu, -B) * dh_of(ph), (phn - ph) / P.dt, S);       // sum c_a h'_a d_t phi_a [A12]
    Q = fma(h, fma(-2.0 * P.A1[a], mu, -P.B1[a]) * P.dTdt, Q);              // sum h_a dc_a/dT d_t T
  }
  md[c] = fma(P.dt, (div - S - Q) / chi, mu);
}

}  // namespace p2

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
static p2::Params g_dummy;  // (size reference for the binding)

void p2_fill_params(const pf_params& p, int liquid, void* out) {
  p2::Params& P = *reinterpret_cast<p2::Params*>(out);
  P = p2::Params{};
  P.dx = p.dx;
  P.dt = p.dt;
  P.eps = p.eps;
  P.inv_dx = 1.0 / p.dx;
  P.dt_over_eps = p.dt / p.eps;
  P.at_c = M_PI * p.eps / 4.0;
  P.dTdt = -p.G * p.v;
  P.Tdz = p.G * p.dx;
  double tsum = 0.0;
  int np = 0;
  for (int a = 0; a < 3; ++a) {
    for (int b = 0; b < 3; ++b) {
      P.g[a][b] = a == b ? 0.0 : p.gamma[a][b];
      P.og[a][b] = a == b ? 0.0 : 16.0 / (M_PI * M_PI) * p.gamma[a][b];
      P.tau[a][b] = p.tau[a][b];
      P.delta[a][b] = p.aniso ? p.aniso_delta[a][b] : 0.0;
      for (int i = 0; i < 9; ++i) P.R[a][b][i] = p.aniso ? p.aniso_R[a][b][i / 3][i % 3] : (i % 4 == 0 ? 1.0 : 0.0);
      if (b > a) {
        tsum += p.tau[a][b];
        ++np;
      }
    }
    P.A0[a] = p.A0[a][0][0];
    P.A1[a] = p.A1[a][0][0];
    P.B0[a] = p.B0[a][0];
    P.B1[a] = p.B1[a][0];
    P.C0[a] = p.C0[a];
    P.C1[a] = p.C1[a];
    P.D[a] = p.D[a][0][0];
  }
  P.g3 = p.gamma3[0][1][2];
  P.inv_tau_mean = np / tsum;
  P.liquid = liquid;
  P.aniso = p.aniso ? 1 : 0;
  P.mu_inf = p.mu_inf[0];
}
size_t p2_params_size() { return sizeof(g_dummy); }

void p2_launch_phi(const void* Pv, double Tbase, const Geom& g, const double* ps, const double* ms, double* pd,
                   cudaStream_t s) {
  p2::Params P = *reinterpret_cast<const p2::Params*>(Pv);
  P.Tbase = Tbase;
  dim3 b(32, 4, 2), gr((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  p2::k_phi<<<gr, b, 0, s>>>(P, g, ps, ms, pd);
}

void p2_launch_mu(const void* Pv, double Tbase, const Geom& g, const double* ps, const double* pd, const double* ms,
                  double* md, cudaStream_t s) {
  p2::Params P = *reinterpret_cast<const p2::Params*>(Pv);
  P.Tbase = Tbase;
  dim3 b(32, 4, 2), gr((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  p2::k_mu<<<gr, b, 0, s>>>(P, g, ps, pd, ms, md);
}

}  // namespace pf
