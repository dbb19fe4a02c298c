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
// Kernels (pf_tuning p2_phi / p2_mu, tuned by pf_autotune): side-staged
// z-marching sweeps (default; k_phi_side, k_mu_side: every face flux
// evaluated once, both sides of a face from shared memory), z-marching
// sweeps that load the face operands from global memory (k_phi_march,
// k_mu_march), and one thread per cell with every face evaluated by both of
// its cells (k_phi, k_mu: the paper's "full" kernels).  Written from the paper;
// parity against the oracle in tests/test_gpu_p2.py.
// Independent of oracle/ (no shared code).
#include <math.h>

#include "pf_internal.h"

namespace pf {
namespace p2 {

constexpr int N3 = 3, NS = 2;  // phases, solids

struct Params {
  double dx, dt, eps, inv_eps, inv_dx, inv_dt, dt_over_eps, at_c, dTdt, Tbase, Tdz;
  double g[N3][N3], og[N3][N3];  // gamma_ab, 16/pi^2 gamma_ab
  double g3;                     // gamma_012
  double tau[N3][N3], inv_tau_mean;
  double A0[N3], A1[N3], B0[N3], B1[N3], C0[N3], C1[N3];  // psi_a = A mu^2 + B mu + C (M = 1), affine in T
  double D[N3];
  double delta[N3][N3];
  double R[N3][N3][9];  // R_ab row-major
  int liquid, aniso;
  int prefetch;  // z-marching sweeps: own column's lines P2_PD planes ahead into L2 (PF_P2_PREFETCH, default 1)
  int side_pd;   // side-staged sweeps: L2 prefetch distance in planes, 0 = off (pf_tuning p2_pd)
  double mu_inf;
};

// 1/x and 1/sqrt(x) for normal x > 0: hardware approximation + one
// third-order Newton step (<= 1 / 2 ulp, reading A18; as pf_model.cuh)
__device__ __forceinline__ double rcp_nr(double x) {
  double y;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  const double e = fma(-x, y, 1.0);
  return fma(y, fma(e, e, e), y);
}
__device__ __forceinline__ double rsqrt_nr(double x) {
  double y;
  asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  const double e = fma(-x * y, y, 1.0);
  return fma(y * e, fma(0.375, e, 0.5), y);
}

__device__ __forceinline__ double h_of(double x) { return x * x * (3.0 - 2.0 * x); }
__device__ __forceinline__ double dh_of(double x) { return 6.0 * x * (1.0 - x); }

// grad_q f, f(q) = A(R q)^2 |q|^2 (reading B6); 0 at q = 0 (f is C^1 there)
__device__ __forceinline__ void aniso_grad(const Params& P, int a, int b, const double q[3], double out[3]) {
  const double* R = P.R[a][b];
  const double delta = P.delta[a][b];
  double v[3];
#pragma unroll
  for (int i = 0; i < 3; ++i) v[i] = fma(R[3 * i], q[0], fma(R[3 * i + 1], q[1], R[3 * i + 2] * q[2]));
  double n2 = fma(v[0], v[0], fma(v[1], v[1], v[2] * v[2]));
  if (n2 == 0.0) {
    out[0] = out[1] = out[2] = 0.0;
    return;
  }
  // below 1e-280 the approximate reciprocal of n2^2 would flush to zero:
  // scale p by 2^300 (exact); A is homogeneous of degree 0 and grad_p f of
  // degree 1, so the result is scaled back by 2^-300
  const bool tiny = n2 < 1e-280;
  const double sc = tiny ? 0x1p300 : 1.0, two_sc = tiny ? 0x1p-299 : 2.0;  // two_sc = 2 / sc (exact)
#pragma unroll
  for (int i = 0; i < 3; ++i) v[i] *= sc;
  n2 *= sc * sc;
  double s4 = 0.0;
#pragma unroll
  for (int i = 0; i < 3; ++i) s4 = fma(v[i] * v[i], v[i] * v[i], s4);
  const double i2 = rcp_nr(n2), i4 = i2 * i2;
  const double A = 1.0 - delta * (3.0 - 4.0 * s4 * i4);
  // dA/dp_i n2 = 16 delta (p_i^3 / n2 - s4 p_i / n2^2)
  double gp[3];
#pragma unroll
  for (int i = 0; i < 3; ++i) {
    const double dAn2 = 16.0 * delta * v[i] * fma(v[i] * v[i], i2, -s4 * i4);
    gp[i] = two_sc * A * fma(A, v[i], dAn2);
  }
#pragma unroll
  for (int j = 0; j < 3; ++j) out[j] = fma(R[j], gp[0], fma(R[3 + j], gp[1], R[6 + j] * gp[2]));
}

// staggered phi flux (d-component of d a / d grad phi_a) at a face in
// direction d from its operands: pb = mean phi, G = face gradient (normal
// difference, means of the tangential central differences)
__device__ __forceinline__ void phi_flux(const Params& P, int d, const double (&pb)[N3], const double (&G)[N3][3],
                                         double j[N3]) {
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

// phi flux at the face p | p+e_d with its operands loaded from global memory;
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
  phi_flux(P, d, pb, G, j);
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

// phi cell update (C.1 S2 steps 2-8) at plane z from its operands: phi,
// the raw central differences cd[b][d] = phi_b(+e_d) - phi_b(-e_d), mu and
// the flux divergence div (eq. 11); out = phi_dst
__device__ __forceinline__ void phi_cell_v(const Params& P, int z, const double (&ph)[N3], const double (&cd)[N3][3],
                                           double mu, const double (&div)[N3], double (&out)[N3]) {
  // 2. cell-centred gradients (central differences) [A10]
  double gd[N3][3];
#pragma unroll
  for (int b = 0; b < N3; ++b)
#pragma unroll
    for (int d = 0; d < 3; ++d) gd[b][d] = cd[b][d] * (0.5 * P.inv_dx);
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
    r[a] = fma(P.eps, dad[a] - div[a], fma(om, P.inv_eps, psi * dh_of(ph[a])));
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
  const double f = den != 0.0 ? P.dt_over_eps * (den * rcp_nr(num)) : P.dt_over_eps * P.inv_tau_mean;
  const double rbar = (r[0] + r[1] + r[2]) * (1.0 / 3.0);
#pragma unroll
  for (int a = 0; a < N3; ++a) out[a] = fma(f, rbar - r[a], ph[a]);
  project3(out);
}
// phi cell update of cell c at plane z with its operands loaded from global memory
__device__ __forceinline__ void phi_cell(const Params& P, const Geom& g, const double* __restrict__ ps,
                                         const double* __restrict__ ms, double* __restrict__ pd, i64 c, int z,
                                         const double (&div)[N3]) {
  const i64 F = g.field;
  const i64 st[3] = {1, g.pitch, g.plane};
  double ph[N3], cd[N3][3], out[N3];
#pragma unroll
  for (int a = 0; a < N3; ++a) ph[a] = __ldg(ps + a * F + c);
#pragma unroll
  for (int b = 0; b < N3; ++b)
#pragma unroll
    for (int d = 0; d < 3; ++d) cd[b][d] = __ldg(ps + b * F + c + st[d]) - __ldg(ps + b * F + c - st[d]);
  phi_cell_v(P, z, ph, cd, __ldg(ms + c), div, out);
#pragma unroll
  for (int a = 0; a < N3; ++a) pd[a * F + c] = out[a];
}

// one thread per cell, every face evaluated by both of its cells
__global__ void __launch_bounds__(256) k_phi(Params P, Geom g, const double* __restrict__ ps,
                                             const double* __restrict__ ms, double* __restrict__ pd) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const i64 c = g.at(x, y, z), F = g.field;
  const i64 st[3] = {1, g.pitch, g.plane};
  double div[N3] = {0.0, 0.0, 0.0};
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    double jp[N3], jm[N3];
    phi_face(P, ps, F, c, d, st, jp);
    phi_face(P, ps, F, c - st[d], d, st, jm);
#pragma unroll
    for (int a = 0; a < N3; ++a) div[a] += (jp[a] - jm[a]) * P.inv_dx;
  }
  phi_cell(P, g, ps, ms, pd, c, z, div);
}

// mu flux F = M grad mu - J_at at a face in direction d (eqs. 8-10)
// [A7-A11], M = 1, from the face operands: pb = mean phi, G = face gradient
// (normal difference, means of the tangential central differences), dtp =
// mean d_t phi, mb / dmu = mean / normal difference of mu
template <int L>
__device__ __forceinline__ double mu_flux(const Params& P, int d, const double (&pb)[N3], const double (&G)[N3][3],
                                          const double (&dtp)[N3], double mb, double dmu, double Tf) {
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
    // g h_l / sqrt(pb_a pb_l) (n_a . n_l) n_a,d = pb_a h_l (G_a . G_l) G_a,d / sqrt(pb_a pb_l nl2 na2^2):
    // one reciprocal square root per solid (as the P1 mu_face)
    const double dot = fma(G[a][0], G[L][0], fma(G[a][1], G[L][1], G[a][2] * G[L][2]));
    const double w = P.at_c * h_of(pb[L]) * dtp[a] * pb[a] * rsqrt_nr(pb[a] * pb[L] * nl2 * na2 * na2);
    const double ca = fma(-2.0 * fma(P.A1[a], Tf, P.A0[a]), mb, -fma(P.B1[a], Tf, P.B0[a]));
    Fl -= w * (cl - ca) * (dot * G[a][d]);
  }
  return Fl;
}

// mu flux at the face p | p+e_d with its operands loaded from global memory
template <int L>
__device__ __forceinline__ double mu_face(const Params& P, const double* __restrict__ ps,
                                          const double* __restrict__ pd, const double* __restrict__ ms, i64 F, i64 c,
                                          int d, const i64 st[3], double Tf) {
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
    dtp[a] = ((__ldg(pd + a * F + c) - vp) + (__ldg(pd + a * F + c + sn) - vq)) * (0.5 * P.inv_dt);
  }
  const double mp = __ldg(ms + c), mq = __ldg(ms + c + sn);
  return mu_flux<L>(P, d, pb, G, dtp, 0.5 * (mp + mq), (mq - mp) * P.inv_dx, Tf);
}

// mu cell update (C.1 S4 steps 2-3, eq. 8) of cell c at plane z given div
// from mu, phi and dphi = phi_dst - phi_src of the cell
__device__ __forceinline__ double mu_cell_v(const Params& P, int z, double mu, const double (&ph)[N3],
                                            const double (&dph)[N3], double div) {
  const double T = fma(P.Tdz, (double)z, P.Tbase);
  double chi = 0.0, S = 0.0, Q = 0.0;
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    const double A = fma(P.A1[a], T, P.A0[a]), B = fma(P.B1[a], T, P.B0[a]);
    const double h = h_of(ph[a]);
    chi = fma(h, -2.0 * A, chi);                                            // chi = sum h_a chi_a
    S = fma(fma(-2.0 * A, mu, -B) * dh_of(ph[a]), dph[a] * P.inv_dt, S);  // sum c_a h'_a d_t phi_a [A12]
    Q = fma(h, fma(-2.0 * P.A1[a], mu, -P.B1[a]) * P.dTdt, Q);              // sum h_a dc_a/dT d_t T
  }
  return fma(P.dt * rcp_nr(chi), div - S - Q, mu);
}
__device__ __forceinline__ void mu_cell(const Params& P, const Geom& g, const double* __restrict__ ps,
                                        const double* __restrict__ pd, const double* __restrict__ ms,
                                        double* __restrict__ md, i64 c, int z, double div) {
  const i64 F = g.field;
  double ph[N3], dph[N3];
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    ph[a] = __ldg(ps + a * F + c);
    dph[a] = __ldg(pd + a * F + c) - ph[a];
  }
  md[c] = mu_cell_v(P, z, __ldg(ms + c), ph, dph, div);
}

template <int L>
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
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    const double Tp = d == 2 ? fma(P.Tdz, z + 0.5, P.Tbase) : T, Tm = d == 2 ? fma(P.Tdz, z - 0.5, P.Tbase) : T;
    div += (mu_face<L>(P, ps, pd, ms, F, c, d, st, Tp) - mu_face<L>(P, ps, pd, ms, F, c - st[d], d, st, Tm)) *
           P.inv_dx;
  }
  mu_cell(P, g, ps, pd, ms, md, c, z, div);
}

// ---------------------------------------------------------------------------
// z-marching sweeps: a CTA owns a TXP x TYP column tile and marches a z-chunk;
// every face flux is evaluated once: each thread the -x, -y and +z faces of
// its cell (the -z face is the previous plane's +z, in registers), the +x
// face from the next lane (shuffle), the +y face from the next row (shared
// memory, double-buffered by plane parity: one barrier per plane), the tile's
// far edges by one extra warp each.  Same face and cell arithmetic as the
// one-thread-per-cell kernels, so the same bits.
// ---------------------------------------------------------------------------
constexpr int TXP = 32, TYP = 4, ZCP = 16;


__device__ __forceinline__ void pf_l2(const double* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }

// own column's lines of the fields a sweep reads, PD planes ahead, into L2
constexpr int P2_PD = 3;

template <int K, class FaceF, class CellF, class PrefF>
__device__ __forceinline__ void march(const Geom& g, bool prefetch, FaceF face, CellF cell, PrefF pref) {
  __shared__ double fy[2][K][TYP][TXP];  // -y face flux of every thread
  __shared__ double ex[2][K][TYP];       // +x flux on the right tile edge
  __shared__ double ey[2][K][TXP];       // +y flux on the top tile edge
  const int lane = threadIdx.x, w = threadIdx.y;
  const int x0 = blockIdx.x * TXP, y0 = blockIdx.y * TYP;
  const int x = x0 + lane, y = y0 + w;
  const bool active = x < g.nx && y < g.ny;
  // ragged tiles: clamp to the ghost cell, whose -x / -y face is the +x / +y
  // face of the last interior cell
  const int xc = min(x, g.nx), yc = min(y, g.ny);
  const int z0 = blockIdx.z * ZCP, z1 = min(z0 + ZCP, g.nz);
  const bool xe = w == 0 && lane < TYP, ye = w == 1;
  const int exc = min(x0 + TXP - 1, g.nx), eyc = min(y0 + TYP - 1, g.ny);
  double Fzm[K];
  face(g.at(xc, yc, z0 - 1), 2, z0 - 1, Fzm);
#pragma unroll 1
  for (int z = z0; z < z1; ++z) {
    const int b = z & 1;
    const i64 c = g.at(xc, yc, z);
    if (prefetch && z + P2_PD <= z1) pref(c + P2_PD * g.plane);
    double Fx[K], Fy[K], Fzp[K];
    face(c - 1, 0, z, Fx);
    face(c - g.pitch, 1, z, Fy);
    face(c, 2, z, Fzp);
    if (xe) {
      double fe[K];
      face(g.at(exc, min(y0 + lane, g.ny), z), 0, z, fe);
#pragma unroll
      for (int a = 0; a < K; ++a) ex[b][a][lane] = fe[a];
    } else if (ye) {
      double fe[K];
      face(g.at(min(x0 + lane, g.nx), eyc, z), 1, z, fe);
#pragma unroll
      for (int a = 0; a < K; ++a) ey[b][a][lane] = fe[a];
    }
#pragma unroll
    for (int a = 0; a < K; ++a) fy[b][a][w][lane] = Fy[a];
    __syncthreads();
    double div[K];
#pragma unroll
    for (int a = 0; a < K; ++a) {
      double fxp = __shfl_down_sync(0xffffffffu, Fx[a], 1);
      if (lane == TXP - 1) fxp = ex[b][a][w];
      const double fyp = w < TYP - 1 ? fy[b][a][w + 1][lane] : ey[b][a][lane];
      div[a] = (fxp - Fx[a]) + (fyp - Fy[a]) + (Fzp[a] - Fzm[a]);
    }
    if (active) cell(c, z, div);
#pragma unroll
    for (int a = 0; a < K; ++a) Fzm[a] = Fzp[a];
  }
}

// MB: CTAs per SM the kernel is compiled for (register cap 65536 / (128 MB))
template <int MB>
__global__ void __launch_bounds__(TXP * TYP, MB) k_phi_march(Params P, Geom g, const double* __restrict__ ps,
                                                         const double* __restrict__ ms, double* __restrict__ pd) {
  const i64 F = g.field;
  const i64 st[3] = {1, g.pitch, g.plane};
  march<N3>(
      g, P.prefetch != 0, [&](i64 c, int d, int, double* j) { phi_face(P, ps, F, c, d, st, j); },
      [&](i64 c, int z, const double* dv) {
        double div[N3];
#pragma unroll
        for (int a = 0; a < N3; ++a) div[a] = dv[a] * P.inv_dx;
        phi_cell(P, g, ps, ms, pd, c, z, div);
      },
      [&](i64 cp) {
#pragma unroll
        for (int a = 0; a < N3; ++a) pf_l2(ps + a * F + cp);
        pf_l2(ms + cp);
      });
}

template <int L, int MB>
__global__ void __launch_bounds__(TXP * TYP, MB) k_mu_march(Params P, Geom g, const double* __restrict__ ps,
                                                        const double* __restrict__ pd, const double* __restrict__ ms,
                                                        double* __restrict__ md) {
  const i64 F = g.field;
  const i64 st[3] = {1, g.pitch, g.plane};
  march<1>(
      g, P.prefetch != 0,
      [&](i64 c, int d, int z, double* f) {
        // T at the face: plane z for x / y faces, z + 1/2 for the face z | z+1 [A13]
        const double Tf = fma(P.Tdz, d == 2 ? z + 0.5 : (double)z, P.Tbase);
        f[0] = mu_face<L>(P, ps, pd, ms, F, c, d, st, Tf);
      },
      [&](i64 c, int z, const double* dv) { mu_cell(P, g, ps, pd, ms, md, c, z, dv[0] * P.inv_dx); },
      [&](i64 cp) {
#pragma unroll
        for (int a = 0; a < N3; ++a) {
          pf_l2(ps + a * F + cp);
          pf_l2(pd + a * F + cp);
        }
        pf_l2(ms + cp);
      });
}

// ---------------------------------------------------------------------------
// mu-sweep with the face operands staged in shared memory (default; the
// z-marching k_mu_march above with PF_P2_MU=march).  A CTA of 32 x TYS
// threads owns a 32 x TYS column tile and marches a z-chunk; per plane k
// every cell of the tile and of its one-cell halo ring publishes its side
//   S = (phi, cd_x, cd_y, cd_z, dphi = phi_dst - phi_src, mu)
// to shared memory once (an own cell loads 14 values, its z column carried
// in registers; a halo cell 19), the -x / -y faces of plane k read both
// sides from there, the z-face k-1 | k pairs the own side of plane k-1
// (registers) with that of plane k, and the cell update of plane k-1 follows
// it (one-plane lag, as the P1 mu-sweep).  The faces' operands are the same
// differences as mu_face's loads, through the same mu_flux: same bits.
// ---------------------------------------------------------------------------
constexpr int TYS = 8, ZCS = 16;  // default tile height (PF_P2_SIDE selects others)
constexpr int SHX = TXP + 2;       // halo-tile row length (a tile of height TY has SHX (TY + 2) cells)
// shared side layout, component-major [SV][SN] (a warp's reads are contiguous)
constexpr int S_F = 0, S_CX = 3, S_CY = 6, S_CZ = 9, S_DP = 12, S_MU = 15, SV = 16;
__device__ __forceinline__ int sidx(int hx, int hy) { return hy * SHX + hx; }

struct Side {
  double f[N3], c1[N3], c2[N3], dp[N3], m;  // c1 / c2: central differences along the two tangential axes
};
template <int SN>
__device__ __forceinline__ void side_ld(const double (*S)[SN], int i, int o1, int o2, Side& s) {
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    s.f[a] = S[S_F + a][i];
    s.c1[a] = S[o1 + a][i];
    s.c2[a] = S[o2 + a][i];
    s.dp[a] = S[S_DP + a][i];
  }
  s.m = S[S_MU][i];
}
// flux at the face p | q in direction d (tangential axes in ascending order in c1, c2)
template <int L>
__device__ __forceinline__ double mu_face_side(const Params& P, int d, const Side& p, const Side& q, double Tf) {
  double pb[N3], G[N3][3], dtp[N3];
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    pb[a] = 0.5 * (p.f[a] + q.f[a]);
    const double gn = (q.f[a] - p.f[a]) * P.inv_dx;
    const double t1 = (p.c1[a] + q.c1[a]) * (0.25 * P.inv_dx), t2 = (p.c2[a] + q.c2[a]) * (0.25 * P.inv_dx);
    G[a][0] = d == 0 ? gn : t1;
    G[a][1] = d == 1 ? gn : (d == 0 ? t1 : t2);
    G[a][2] = d == 2 ? gn : t2;
    dtp[a] = (p.dp[a] + q.dp[a]) * (0.5 * P.inv_dt);
  }
  return mu_flux<L>(P, d, pb, G, dtp, 0.5 * (p.m + q.m), (q.m - p.m) * P.inv_dx, Tf);
}

template <int L, int TY, int MB>
__global__ void __launch_bounds__(TXP * TY, MB) k_mu_side(Params P, Geom g, const double* __restrict__ ps,
                                                         const double* __restrict__ pd,
                                                         const double* __restrict__ ms, double* __restrict__ md) {
  constexpr int SN = SHX * (TY + 2);
  __shared__ double S[SV][SN];
  __shared__ double fxs[TY][TXP + 1];  // -x flux of every cell, +x of the right tile edge at TXP
  __shared__ double fys[TY + 1][TXP];  // -y flux of every cell, +y of the top tile edge at TY
  const i64 F = g.field;
  const int lane = threadIdx.x, w = threadIdx.y, t = w * TXP + lane;
  constexpr int NT = TXP * TY;
  const int x0 = blockIdx.x * TXP, y0 = blockIdx.y * TY;
  const int x = x0 + lane, y = y0 + w;
  const bool active = x < g.nx && y < g.ny;
  const int xc = min(x, g.nx), yc = min(y, g.ny);
  const int me = sidx(lane + 1, w + 1);
  const int z0 = blockIdx.z * ZCS, z1 = min(z0 + ZCS, g.nz);
  // halo ring: the last 2 TXP + 2 TY threads, one cell each (columns first)
  const int th = t - (NT - 2 * TXP - 2 * TY);
  int hx = 0, hy = 0;
  bool hcol = false;
  if (th >= 0 && th < 2 * TY) {
    hcol = true;
    hx = th < TY ? 0 : TXP + 1;
    hy = (th < TY ? th : th - TY) + 1;
  } else if (th >= 2 * TY) {
    const int r = th - 2 * TY;
    hx = (r < TXP ? r : r - TXP) + 1;
    hy = r < TXP ? 0 : TY + 1;
  }
  const int hs = th >= 0 ? sidx(hx, hy) : -1;
  const i64 hoff = th >= 0 ? g.at(min(x0 + hx - 1, g.nx), min(y0 + hy - 1, g.ny), 0) : 0;
  const i64 htan = hcol ? g.pitch : 1;  // the halo cell's in-plane tangential axis (y for columns, x for rows)
  const i64 coff = g.at(xc, yc, 0);

  // own side of plane z0 - 1 (z-face operands: f, cd_x, cd_y, dphi, mu) and the carried phi column
  Side Sp;
  double fc[N3], fm[N3];
  const bool pfl = (lane & 15) == 0 || th >= 0;  // one L2 prefetch per 128-B line of the own rows; halo cells
  const i64 pfo = th >= 0 ? hoff : coff;
  {
    const i64 c = coff + (i64)(z0 - 1) * g.plane;
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      const double* f = ps + a * F + c;
      Sp.f[a] = __ldg(f);
      Sp.c1[a] = __ldg(f + 1) - __ldg(f - 1);
      Sp.c2[a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
      Sp.dp[a] = __ldg(pd + a * F + c) - Sp.f[a];
      fm[a] = Sp.f[a];
      fc[a] = __ldg(f + g.plane);
    }
    Sp.m = __ldg(ms + c);
  }
  double divxy = 0.0, Fzm = 0.0;
  for (int k = z0; k <= z1; ++k) {
    const bool last = k == z1;
    const i64 c = coff + (i64)k * g.plane;
    if (P.side_pd && pfl && k + P.side_pd <= z1) {
      const i64 cp = pfo + (i64)(k + P.side_pd) * g.plane;
#pragma unroll
      for (int a = 0; a < N3; ++a) {
        pf_l2(ps + a * F + cp);
        pf_l2(pd + a * F + cp);
      }
      pf_l2(ms + cp);
    }
    // (a) publish the sides of plane k
    Side Q;  // own side, tangential (x, y) for the z-face
    double cz[N3];
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      const double* f = ps + a * F + c;
      const double fp = !last ? __ldg(f + g.plane) : 0.0;
      Q.f[a] = fc[a];
      Q.c1[a] = __ldg(f + 1) - __ldg(f - 1);
      Q.c2[a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
      cz[a] = !last ? fp - fm[a] : 0.0;
      Q.dp[a] = __ldg(pd + a * F + c) - fc[a];
      fm[a] = fc[a];
      fc[a] = fp;
    }
    Q.m = __ldg(ms + c);
    if (!last) {
#pragma unroll
      for (int a = 0; a < N3; ++a) {
        S[S_F + a][me] = Q.f[a];
        S[S_CX + a][me] = Q.c1[a];
        S[S_CY + a][me] = Q.c2[a];
        S[S_CZ + a][me] = cz[a];
        S[S_DP + a][me] = Q.dp[a];
      }
      S[S_MU][me] = Q.m;
      if (hs >= 0) {
        const i64 ch = hoff + (i64)k * g.plane;
#pragma unroll
        for (int a = 0; a < N3; ++a) {
          const double* f = ps + a * F + ch;
          const double v = __ldg(f), tt = __ldg(f + htan) - __ldg(f - htan);
          S[S_F + a][hs] = v;
          S[S_CX + a][hs] = hcol ? 0.0 : tt;
          S[S_CY + a][hs] = hcol ? tt : 0.0;
          S[S_CZ + a][hs] = __ldg(f + g.plane) - __ldg(f - g.plane);
          S[S_DP + a][hs] = __ldg(pd + a * F + ch) - v;
        }
        S[S_MU][hs] = __ldg(ms + ch);
      }
    }
    __syncthreads();
    // (b) z-face k-1 | k and (c) the cell update of plane k-1
    const double Fz = mu_face_side<L>(P, 2, Sp, Q, fma(P.Tdz, (k - 1) + 0.5, P.Tbase));
    if (k > z0 && active) {
      const double div = divxy + (Fz - Fzm);
      md[c - g.plane] = mu_cell_v(P, k - 1, Sp.m, Sp.f, Sp.dp, div * P.inv_dx);
    }
    Fzm = Fz;
    if (last) break;
    // (d) x / y faces of plane k: -x and -y of every cell, + the far tile edges
    const double Tk = fma(P.Tdz, (double)k, P.Tbase);
    Side p, q;
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      q.f[a] = Q.f[a];
      q.c1[a] = Q.c2[a];  // tangential y, z
      q.c2[a] = cz[a];
      q.dp[a] = Q.dp[a];
    }
    q.m = Q.m;
    side_ld(S, me - 1, S_CY, S_CZ, p);
    const double Fx = mu_face_side<L>(P, 0, p, q, Tk);
#pragma unroll
    for (int a = 0; a < N3; ++a) q.c1[a] = Q.c1[a];  // tangential x, z
    side_ld(S, me - SHX, S_CX, S_CZ, p);
    const double Fy = mu_face_side<L>(P, 1, p, q, Tk);
    fxs[w][lane] = Fx;
    fys[w][lane] = Fy;
    if (w == 0 && lane < TY) {  // +x face of the right tile edge, row `lane`
      side_ld(S, sidx(TXP, lane + 1), S_CY, S_CZ, p);
      side_ld(S, sidx(TXP + 1, lane + 1), S_CY, S_CZ, q);
      fxs[lane][TXP] = mu_face_side<L>(P, 0, p, q, Tk);
    } else if (w == 1) {  // +y face of the top tile edge, column `lane`
      side_ld(S, sidx(lane + 1, TY), S_CX, S_CZ, p);
      side_ld(S, sidx(lane + 1, TY + 1), S_CX, S_CZ, q);
      fys[TY][lane] = mu_face_side<L>(P, 1, p, q, Tk);
    }
    __syncthreads();
    divxy = (fxs[w][lane + 1] - Fx) + (fys[w + 1][lane] - Fy);
#pragma unroll
    for (int a = 0; a < N3; ++a) Sp.f[a] = Q.f[a], Sp.c1[a] = Q.c1[a], Sp.c2[a] = Q.c2[a], Sp.dp[a] = Q.dp[a];
    Sp.m = Q.m;
  }
}

// ---------------------------------------------------------------------------
// phi-sweep with the face operands staged in shared memory (default;
// k_phi_march with PF_P2_PHI=march): the scheme of k_mu_side with
// the side (phi, cd_x, cd_y, cd_z) and three fluxes per face; the cell update
// takes phi, the central differences and mu of the own cell from registers.
// ---------------------------------------------------------------------------
constexpr int P_F = 0, P_CX = 3, P_CY = 6, P_CZ = 9, PV = 12;
struct PSide {
  double f[N3], c1[N3], c2[N3];
};
template <int SN>
__device__ __forceinline__ void pside_ld(const double (*S)[SN], int i, int o1, int o2, PSide& s) {
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    s.f[a] = S[P_F + a][i];
    s.c1[a] = S[o1 + a][i];
    s.c2[a] = S[o2 + a][i];
  }
}
__device__ __forceinline__ void phi_face_side(const Params& P, int d, const PSide& p, const PSide& q, double j[N3]) {
  double pb[N3], G[N3][3];
#pragma unroll
  for (int a = 0; a < N3; ++a) {
    pb[a] = 0.5 * (p.f[a] + q.f[a]);
    const double gn = (q.f[a] - p.f[a]) * P.inv_dx;
    const double t1 = (p.c1[a] + q.c1[a]) * (0.25 * P.inv_dx), t2 = (p.c2[a] + q.c2[a]) * (0.25 * P.inv_dx);
    G[a][0] = d == 0 ? gn : t1;
    G[a][1] = d == 1 ? gn : (d == 0 ? t1 : t2);
    G[a][2] = d == 2 ? gn : t2;
  }
  phi_flux(P, d, pb, G, j);
}

template <int TY, int MB>
__global__ void __launch_bounds__(TXP * TY, MB) k_phi_side(Params P, Geom g, const double* __restrict__ ps,
                                                          const double* __restrict__ ms, double* __restrict__ pd) {
  constexpr int SN = SHX * (TY + 2);
  __shared__ double S[PV][SN];
  __shared__ double fxs[N3][TY][TXP + 1];
  __shared__ double fys[N3][TY + 1][TXP];
  const i64 F = g.field;
  const int lane = threadIdx.x, w = threadIdx.y, t = w * TXP + lane;
  constexpr int NT = TXP * TY;
  const int x0 = blockIdx.x * TXP, y0 = blockIdx.y * TY;
  const int x = x0 + lane, y = y0 + w;
  const bool active = x < g.nx && y < g.ny;
  const int xc = min(x, g.nx), yc = min(y, g.ny);
  const int me = sidx(lane + 1, w + 1);
  const int z0 = blockIdx.z * ZCS, z1 = min(z0 + ZCS, g.nz);
  const int th = t - (NT - 2 * TXP - 2 * TY);
  int hx = 0, hy = 0;
  bool hcol = false;
  if (th >= 0 && th < 2 * TY) {
    hcol = true;
    hx = th < TY ? 0 : TXP + 1;
    hy = (th < TY ? th : th - TY) + 1;
  } else if (th >= 2 * TY) {
    const int r = th - 2 * TY;
    hx = (r < TXP ? r : r - TXP) + 1;
    hy = r < TXP ? 0 : TY + 1;
  }
  const int hs = th >= 0 ? sidx(hx, hy) : -1;
  const i64 hoff = th >= 0 ? g.at(min(x0 + hx - 1, g.nx), min(y0 + hy - 1, g.ny), 0) : 0;
  const i64 htan = hcol ? g.pitch : 1;
  const i64 coff = g.at(xc, yc, 0);
  const bool pfl = (lane & 15) == 0 || th >= 0;
  const i64 pfo = th >= 0 ? hoff : coff;

  // own side of plane z0 - 1 (f, cd_x, cd_y, cd_z: z-face and cell operands), mu, carried phi column
  double Sf[N3], Sx[N3], Sy[N3], Sz[N3], Smu;
  double fc[N3], fm[N3];
  {
    const i64 c = coff + (i64)(z0 - 1) * g.plane;
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      const double* f = ps + a * F + c;
      Sf[a] = __ldg(f);
      Sx[a] = __ldg(f + 1) - __ldg(f - 1);
      Sy[a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
      Sz[a] = 0.0;  // (plane z0 - 1 is never updated here)
      fm[a] = Sf[a];
      fc[a] = __ldg(f + g.plane);
    }
    Smu = 0.0;
  }
  double divxy[N3] = {0.0, 0.0, 0.0}, Fzm[N3] = {0.0, 0.0, 0.0};
  for (int k = z0; k <= z1; ++k) {
    const bool last = k == z1;
    const i64 c = coff + (i64)k * g.plane;
    if (P.side_pd && pfl && k + P.side_pd <= z1) {
      const i64 cp = pfo + (i64)(k + P.side_pd) * g.plane;
#pragma unroll
      for (int a = 0; a < N3; ++a) pf_l2(ps + a * F + cp);
      pf_l2(ms + cp);
    }
    // (a) publish the sides of plane k
    double Qf[N3], Qx[N3], Qy[N3], Qz[N3];
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      const double* f = ps + a * F + c;
      const double fp = !last ? __ldg(f + g.plane) : 0.0;
      Qf[a] = fc[a];
      Qx[a] = __ldg(f + 1) - __ldg(f - 1);
      Qy[a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
      Qz[a] = !last ? fp - fm[a] : 0.0;
      fm[a] = fc[a];
      fc[a] = fp;
    }
    if (!last) {
#pragma unroll
      for (int a = 0; a < N3; ++a) {
        S[P_F + a][me] = Qf[a];
        S[P_CX + a][me] = Qx[a];
        S[P_CY + a][me] = Qy[a];
        S[P_CZ + a][me] = Qz[a];
      }
      if (hs >= 0) {
        const i64 ch = hoff + (i64)k * g.plane;
#pragma unroll
        for (int a = 0; a < N3; ++a) {
          const double* f = ps + a * F + ch;
          const double tt = __ldg(f + htan) - __ldg(f - htan);
          S[P_F + a][hs] = __ldg(f);
          S[P_CX + a][hs] = hcol ? 0.0 : tt;
          S[P_CY + a][hs] = hcol ? tt : 0.0;
          S[P_CZ + a][hs] = __ldg(f + g.plane) - __ldg(f - g.plane);
        }
      }
    }
    __syncthreads();
    // (b) z-face k-1 | k and (c) the cell update of plane k-1
    double Fz[N3];
    {
      PSide p, q;
#pragma unroll
      for (int a = 0; a < N3; ++a) {
        p.f[a] = Sf[a], p.c1[a] = Sx[a], p.c2[a] = Sy[a];
        q.f[a] = Qf[a], q.c1[a] = Qx[a], q.c2[a] = Qy[a];
      }
      phi_face_side(P, 2, p, q, Fz);
    }
    if (k > z0 && active) {
      double div[N3], cd[N3][3], out[N3];
#pragma unroll
      for (int a = 0; a < N3; ++a) {
        div[a] = (divxy[a] + (Fz[a] - Fzm[a])) * P.inv_dx;
        cd[a][0] = Sx[a], cd[a][1] = Sy[a], cd[a][2] = Sz[a];
      }
      phi_cell_v(P, k - 1, Sf, cd, Smu, div, out);
      const i64 cm = c - g.plane;
#pragma unroll
      for (int a = 0; a < N3; ++a) pd[a * F + cm] = out[a];
    }
#pragma unroll
    for (int a = 0; a < N3; ++a) Fzm[a] = Fz[a];
    if (last) break;
    // (d) x / y faces of plane k
    double Fx[N3], Fy[N3];
    {
      PSide p, q;
#pragma unroll
      for (int a = 0; a < N3; ++a) q.f[a] = Qf[a], q.c1[a] = Qy[a], q.c2[a] = Qz[a];
      pside_ld(S, me - 1, P_CY, P_CZ, p);
      phi_face_side(P, 0, p, q, Fx);
#pragma unroll
      for (int a = 0; a < N3; ++a) q.c1[a] = Qx[a];
      pside_ld(S, me - SHX, P_CX, P_CZ, p);
      phi_face_side(P, 1, p, q, Fy);
    }
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      fxs[a][w][lane] = Fx[a];
      fys[a][w][lane] = Fy[a];
    }
    if (w == 0 && lane < TY) {
      PSide p, q;
      double Fe[N3];
      pside_ld(S, sidx(TXP, lane + 1), P_CY, P_CZ, p);
      pside_ld(S, sidx(TXP + 1, lane + 1), P_CY, P_CZ, q);
      phi_face_side(P, 0, p, q, Fe);
#pragma unroll
      for (int a = 0; a < N3; ++a) fxs[a][lane][TXP] = Fe[a];
    } else if (w == 1) {
      PSide p, q;
      double Fe[N3];
      pside_ld(S, sidx(lane + 1, TY), P_CX, P_CZ, p);
      pside_ld(S, sidx(lane + 1, TY + 1), P_CX, P_CZ, q);
      phi_face_side(P, 1, p, q, Fe);
#pragma unroll
      for (int a = 0; a < N3; ++a) fys[a][TY][lane] = Fe[a];
    }
    const double mk = __ldg(ms + c);  // mu of the own cell (plane k), for its update one plane later
    __syncthreads();
#pragma unroll
    for (int a = 0; a < N3; ++a) {
      divxy[a] = (fxs[a][w][lane + 1] - Fx[a]) + (fys[a][w + 1][lane] - Fy[a]);
      Sf[a] = Qf[a], Sx[a] = Qx[a], Sy[a] = Qy[a], Sz[a] = Qz[a];
    }
    Smu = mk;
  }
}

}  // namespace p2

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
void p2_fill_params(const pf_params& p, int liquid, void* out) {
  p2::Params& P = *reinterpret_cast<p2::Params*>(out);
  P = p2::Params{};
  P.dx = p.dx;
  P.dt = p.dt;
  P.eps = p.eps;
  P.inv_dx = 1.0 / p.dx;
  P.inv_dt = 1.0 / p.dt;
  P.inv_eps = 1.0 / p.eps;
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
  const char* e = getenv("PF_P2_PREFETCH");
  P.prefetch = e ? atoi(e) : 1;
  P.side_pd = 2;  // (per launch from P2Cfg)
}
size_t p2_params_size() { return sizeof(p2::Params); }

// CTAs per SM the z-marching kernels are compiled for: 4 (128 registers, a
// 24-64 B spill) by default -- 7.08 vs 6.25 GLUP/s at 256^3 for 3 (168
// registers, no spill), same-box A/B (profiles/r02_ab_p2.json); PF_P2_MINB=3
static int p2_minb() {
  const char* e = getenv("PF_P2_MINB");
  return e && atoi(e) == 3 ? 3 : 4;
}

// Kernel choice (pf_tuning p2_*, P2Cfg): kern 0 = side-staged (default),
// 1 = z-marching with global-memory face operands, 2 = one thread per cell;
// side-staged tile height x CTAs per SM (8, 2) / (8, 1) / (4, 3) / (4, 4),
// measured at 256^3 (profiles/r02_ab_p2.json): phi 1.215 / 2.004 / 1.374 /
// 1.251 ms, mu 0.739 / 1.050 / 0.816 / 0.692 ms (defaults phi (8, 2), mu (4, 4))
void p2_launch_phi(const void* Pv, const P2Cfg& c, double Tbase, const Geom& g, const double* ps, const double* ms,
                   double* pd, cudaStream_t s) {
  p2::Params P = *reinterpret_cast<const p2::Params*>(Pv);
  P.Tbase = Tbase;
  P.side_pd = c.pd;
  if (c.kern == 2) {
    dim3 b(32, 4, 2), gr((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
    p2::k_phi<<<gr, b, 0, s>>>(P, g, ps, ms, pd);
    return;
  }
  if (c.kern == 0) {
    const int ty = c.ty, mb = c.mb;
    dim3 b(p2::TXP, ty), gr((g.nx + p2::TXP - 1) / p2::TXP, (g.ny + ty - 1) / ty, (g.nz + p2::ZCS - 1) / p2::ZCS);
    if (ty == 4 && mb == 3)
      p2::k_phi_side<4, 3><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
    else if (ty == 4)
      p2::k_phi_side<4, 4><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
    else if (mb == 1)
      p2::k_phi_side<8, 1><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
    else
      p2::k_phi_side<8, 2><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
    return;
  }
  dim3 b(p2::TXP, p2::TYP), gr((g.nx + p2::TXP - 1) / p2::TXP, (g.ny + p2::TYP - 1) / p2::TYP,
                               (g.nz + p2::ZCP - 1) / p2::ZCP);
  if (p2_minb() == 4)
    p2::k_phi_march<4><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
  else
    p2::k_phi_march<3><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
}

void p2_launch_mu(const void* Pv, const P2Cfg& c, double Tbase, const Geom& g, const double* ps, const double* pd,
                  const double* ms, double* md, cudaStream_t s) {
  p2::Params P = *reinterpret_cast<const p2::Params*>(Pv);
  P.Tbase = Tbase;
  P.side_pd = c.pd;
  if (c.kern == 2) {
    dim3 b(32, 4, 2), gr((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
    switch (P.liquid) {
      case 0: p2::k_mu<0><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md); break;
      case 1: p2::k_mu<1><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md); break;
      default: p2::k_mu<2><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md); break;
    }
    return;
  }
  if (c.kern == 0) {
    const int ty = c.ty, mb = c.mb;
    dim3 b(p2::TXP, ty), gr((g.nx + p2::TXP - 1) / p2::TXP, (g.ny + ty - 1) / ty, (g.nz + p2::ZCS - 1) / p2::ZCS);
#define PF_P2_MUS(LL)                                                                         \
  (ty == 4 && mb == 3 ? (p2::k_mu_side<LL, 4, 3><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md))     \
   : ty == 4          ? (p2::k_mu_side<LL, 4, 4><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md))     \
   : mb == 1          ? (p2::k_mu_side<LL, 8, 1><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md))     \
                      : (p2::k_mu_side<LL, 8, 2><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md)))
    switch (P.liquid) {
      case 0: PF_P2_MUS(0); break;
      case 1: PF_P2_MUS(1); break;
      default: PF_P2_MUS(2); break;
    }
#undef PF_P2_MUS
    return;
  }
  dim3 b(p2::TXP, p2::TYP), gr((g.nx + p2::TXP - 1) / p2::TXP, (g.ny + p2::TYP - 1) / p2::TYP,
                               (g.nz + p2::ZCP - 1) / p2::ZCP);
#define PF_P2_MU(LL)                                                        \
  (p2_minb() == 4 ? (p2::k_mu_march<LL, 4><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md)) \
                  : (p2::k_mu_march<LL, 3><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md)))
  switch (P.liquid) {  // the liquid index as a compile-time constant (register-resident face arrays)
    case 0: PF_P2_MU(0); break;
    case 1: PF_P2_MU(1); break;
    default: PF_P2_MU(2); break;
  }
#undef PF_P2_MU
}

}  // namespace pf
