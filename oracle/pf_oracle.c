/*
 * pf_oracle.c -- CPU ORACLE (test infrastructure only; see pf_oracle.h).
 *
 * A plain, slow, step-by-step fp64 implementation of one explicit time step
 * of the grand-potential multiphase-field model of Bauer et al. (SC'19),
 * written from the paper in its order and notation:
 *
 *   functional      Psi = int eps*a + omega/eps + psi dV      P:L371-373 (eq. 3)
 *   gradient energy a = sum_{a<b} gamma_ab |q_ab|^2           P:L382-398 (eq. 4)
 *   obstacle        omega                                     P:L400-415 (eq. 5)
 *   grand potential psi_a = mu.A mu + B.mu + C                P:L418-450 (eq. 6)
 *   phi equation    Allen-Cahn + Lagrange multiplier          P:L464-495 (eq. 7)
 *   mu equation     Karma, non-variational                    P:L509-531 (eq. 8)
 *   mobility        M = sum D_a dc_a/dmu g_a                  P:L539-555 (eq. 9)
 *   anti-trapping   J_at                                      P:L556-571 (eq. 10)
 *   discretisation  2nd-order FD, staggered fluxes            P:L590-639 (eq. 11)
 *   time step       Algorithm 1
 *
 * Where the paper is silent or garbled the readings A1..A25 of DESIGN.md §3
 * (= SURVEY.md §8(c)-C.2) are used; each use is marked "[An]".
 *
 * No blocking, no fusion, no caching of face values: every face flux is
 * recomputed from the fields each time a cell needs it (the paper's "full"
 * kernels).  Built with -O2 -ffp-contract=off (no FMA
 * contraction, no fast-math).  Shares no code with the CUDA path.
 */
#include "pf_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define PI_D 3.14159265358979323846

struct pf_oracle {
  or_grid g;
  or_params p;
  int sx, sy, sz;    /* extents including one ghost layer per side */
  double* phi[2];    /* [N][sz][sy][sx] */
  double* mu[2];     /* [M][sz][sy][sx] */
  int cur;           /* src level; dst = 1 - cur */
  or_state st;
};

static int g_threads = 0;
void oracle_set_threads(int n) { g_threads = n < 0 ? 0 : n; }

/* ------------------------------------------------------------------------ */
/* Field access.  Every read of a field goes through rd(), so that the
 * Table-1 footprint pin (P14) can trace which values a cell update loads.    */
/* ------------------------------------------------------------------------ */
enum { F_PHI_SRC = 0, F_PHI_DST = 1, F_MU_SRC = 2, F_FLUX_PHI = 3, F_FLUX_MU = 4 };

#define TRACE_MAX 4096
static struct {
  int on;           /* record reads                                   */
  int virt_flux;    /* face fluxes are read from a (virtual) array    */
  int cx, cy, cz;   /* traced cell                                    */
  int n;
  int key[TRACE_MAX][5];
  int nstore;
} g_tr;

static void trace_read(int f, int comp, int x, int y, int z) {
  int k[5] = {f, comp, x - g_tr.cx, y - g_tr.cy, z - g_tr.cz};
  for (int i = 0; i < g_tr.n; ++i)
    if (!memcmp(g_tr.key[i], k, sizeof k)) return;
  if (g_tr.n < TRACE_MAX) memcpy(g_tr.key[g_tr.n++], k, sizeof k);
}

static inline size_t idx(const pf_oracle* o, int c, int x, int y, int z) {
  /* x, y, z in [-1, n]; c = component */
  return (((size_t)c * o->sz + (size_t)(z + 1)) * o->sy + (size_t)(y + 1)) * o->sx + (size_t)(x + 1);
}

static double rd(const pf_oracle* o, int f, int c, int x, int y, int z) {
  if (g_tr.on) trace_read(f, c, x, y, z);
  switch (f) {
    case F_PHI_SRC: return o->phi[o->cur][idx(o, c, x, y, z)];
    case F_PHI_DST: return o->phi[1 - o->cur][idx(o, c, x, y, z)];
    default: return o->mu[o->cur][idx(o, c, x, y, z)];
  }
}

/* ------------------------------------------------------------------------ */
/* Model functions                                                           */
/* ------------------------------------------------------------------------ */

/* Interpolation h: zero slope at 0 and 1, h(0)=0, h(1)=1 [A4]:
 * h(x) = x^2 (3 - 2x), h'(x) = 6 x (1 - x).  Evaluated in exactly this form
 * so that h(0), h(1), h'(0), h'(1) are exact.                 */
static double h_of(double x) { return x * x * (3.0 - 2.0 * x); }
static double dh_of(double x) { return 6.0 * x * (1.0 - x); }
/* Mobility interpolation g_a = phi_a, "a simpler interpolation" [A4] */
static double g_of(double x) { return x; }

static double gamma3_of(const or_params* p, int a, int b, int d) {
  /* gamma_abd is only defined for a<b<d (eq. 5); read it with sorted indices */
  int s[3] = {a, b, d};
  for (int i = 0; i < 2; ++i)
    for (int j = 0; j < 2 - i; ++j)
      if (s[j] > s[j + 1]) { int t = s[j]; s[j] = s[j + 1]; s[j + 1] = t; }
  return p->gamma3[s[0]][s[1]][s[2]];
}

/* Frozen analytic temperature T(z, t) = T0 + G (z dx - v t), z measured in
 * cells from the origin of the (moving) frame, z = k + z_off (+1/2 on a
 * z-face).  "analytic temperature gradient depending on time and one spatial
 * coordinate" [A13].                                          */
static double temperature(const pf_oracle* o, double zk) {
  double t = (double)o->st.step * o->p.dt;
  return o->p.T0 + o->p.G * ((zk + (double)o->st.z_off) * o->p.dx - o->p.v * t);
}

/* A_a(T), B_a(T), C_a(T) affine in T */
static void coeffs(const or_params* p, int a, double T, double A[OR_MAXM][OR_MAXM],
                   double B[OR_MAXM], double* C) {
  for (int i = 0; i < p->M; ++i) {
    for (int j = 0; j < p->M; ++j) A[i][j] = p->A0[a][i][j] + p->A1[a][i][j] * T;
    B[i] = p->B0[a][i] + p->B1[a][i] * T;
  }
  if (C) *C = p->C0[a] + p->C1[a] * T;
}

/* psi_a(mu, T) = mu . A_a(T) mu + B_a(T) . mu + C_a(T)   (eq. 6) */
static double psi_of(const or_params* p, int a, const double* mu, double T) {
  double A[OR_MAXM][OR_MAXM], B[OR_MAXM], C;
  coeffs(p, a, T, A, B, &C);
  double s = 0.0;
  for (int i = 0; i < p->M; ++i)
    for (int j = 0; j < p->M; ++j) s += mu[i] * A[i][j] * mu[j];
  for (int i = 0; i < p->M; ++i) s += B[i] * mu[i];
  return s + C;
}

/* c_a(mu, T) = -d psi_a / d mu = -(A + A^T) mu - B   [A6]; chi_a = dc_a/dmu = -(A + A^T) */
static void conc_of(const or_params* p, int a, const double* mu, double T, double* c) {
  double A[OR_MAXM][OR_MAXM], B[OR_MAXM];
  coeffs(p, a, T, A, B, NULL);
  for (int i = 0; i < p->M; ++i) {
    double s = 0.0;
    for (int j = 0; j < p->M; ++j) s += (A[i][j] + A[j][i]) * mu[j];
    c[i] = -s - B[i];
  }
}
static void chi_of(const or_params* p, int a, double T, double chi[OR_MAXM][OR_MAXM]) {
  double A[OR_MAXM][OR_MAXM], B[OR_MAXM];
  coeffs(p, a, T, A, B, NULL);
  for (int i = 0; i < p->M; ++i)
    for (int j = 0; j < p->M; ++j) chi[i][j] = -(A[i][j] + A[j][i]);
}
/* dc_a/dT = -(A1 + A1^T) mu - B1 */
static void dcdT_of(const or_params* p, int a, const double* mu, double* out) {
  for (int i = 0; i < p->M; ++i) {
    double s = 0.0;
    for (int j = 0; j < p->M; ++j) s += (p->A1[a][i][j] + p->A1[a][j][i]) * mu[j];
    out[i] = -s - p->B1[a][i];
  }
}

/* Euclidean projection onto the Gibbs simplex {phi >= 0, sum phi = 1} [A14]:
 * sort descending into u; rho = max{j : u_j - (sum_{i<=j} u_i - 1)/j > 0};
 * theta = (sum_{i<=rho} u_i - 1)/rho; out = max(x - theta, 0).               */
void oracle_project_simplex(int N, const double* x, double* out) {
  double u[OR_MAXN];
  for (int i = 0; i < N; ++i) u[i] = x[i];
  for (int i = 0; i < N; ++i) /* plain insertion sort, descending */
    for (int j = i; j > 0 && u[j] > u[j - 1]; --j) { double t = u[j]; u[j] = u[j - 1]; u[j - 1] = t; }
  int rho = 1;
  double s = 0.0, s_rho = u[0];
  for (int j = 1; j <= N; ++j) {
    s += u[j - 1];
    if (u[j - 1] - (s - 1.0) / (double)j > 0.0) { rho = j; s_rho = s; }
  }
  double theta = (s_rho - 1.0) / (double)rho;
  for (int i = 0; i < N; ++i) {
    double y = x[i] - theta;
    out[i] = y > 0.0 ? y : 0.0;
  }
}

/* ------------------------------------------------------------------------ */
/* phi-sweep  (Algorithm 1 line 1)                              */
/* ------------------------------------------------------------------------ */

/* Anisotropic gradient energy (P2, reading B6): f(q) = A(R q)^2 |q|^2 with
 * A(p) = 1 - delta (3 - 4 sum_i p_i^4 / |p|^4).  grad_q f = R^T grad_p f,
 *   d f / d p_i = 2 A (dA/dp_i) |p|^2 + 2 A^2 p_i,
 *   dA/dp_i = 16 delta (p_i^3 / |p|^4 - (sum_j p_j^4) p_i / |p|^6);
 * f -> 0 and grad f -> 0 as q -> 0 (A is bounded): q = 0 gives 0 exactly. */
static void aniso_grad(const or_params* p, int a, int b, const double q[3], double out[3]) {
  const double (*R)[3] = p->aniso_R[a][b];
  const double delta = p->aniso_delta[a][b];
  double v[3];
  for (int i = 0; i < 3; ++i) v[i] = R[i][0] * q[0] + R[i][1] * q[1] + R[i][2] * q[2];
  double n2 = v[0] * v[0] + v[1] * v[1] + v[2] * v[2];
  if (n2 == 0.0) { out[0] = out[1] = out[2] = 0.0; return; }
  double s4 = 0.0;
  for (int i = 0; i < 3; ++i) s4 += v[i] * v[i] * v[i] * v[i];
  double A = 1.0 - delta * (3.0 - 4.0 * s4 / (n2 * n2));
  double gp[3];
  for (int i = 0; i < 3; ++i) {
    double dA = 16.0 * delta * (v[i] * v[i] * v[i] / (n2 * n2) - s4 * v[i] / (n2 * n2 * n2));
    gp[i] = 2.0 * A * dA * n2 + 2.0 * A * A * v[i];
  }
  for (int j = 0; j < 3; ++j) out[j] = R[0][j] * gp[0] + R[1][j] * gp[1] + R[2][j] * gp[2];
}

/* Staggered flux of the gradient energy at the face between p and q = p+e_d
 * (eq. 11 "divergence of fluxes"):
 *   (da/d grad phi_a)_d = 2 sum_{b!=a} gamma_ab phib_b (phib_b d_d phi_a - phib_a d_d phi_b)
 * with q_ab = phi_a grad phi_b - phi_b grad phi_a [A2]; face values are the
 * mean of the two cells, the normal derivative is (phi(q) - phi(p))/dx [A9]. */
static void phi_face_flux(const pf_oracle* o, int x, int y, int z, int d, double* j) {
  const or_params* p = &o->p;
  int qx = x + (d == 0), qy = y + (d == 1), qz = z + (d == 2);
  if (g_tr.on && g_tr.virt_flux) { /* split accounting: the flux is a stored value */
    for (int a = 0; a < p->N; ++a) { trace_read(F_FLUX_PHI, 4 * a + d, x, y, z); j[a] = 0.0; }
    return;
  }
  double pb[OR_MAXN], dd[OR_MAXN];
  for (int b = 0; b < p->N; ++b) {
    double vp = rd(o, F_PHI_SRC, b, x, y, z), vq = rd(o, F_PHI_SRC, b, qx, qy, qz);
    pb[b] = 0.5 * (vp + vq);
    dd[b] = (vq - vp) / p->dx;
  }
  if (p->aniso) {
    /* P2 [B6]: j_a = d a / d (grad phi_a), d-component, at the face:
     * sum_{b != a} gamma_ab (-phib_b) (grad_q f(q_ab))_d with
     * q_ab = phib_a G_b - phib_b G_a and the whole face gradient G (normal
     * difference, tangential = mean of the two central differences [A9]). */
    double G[OR_MAXN][3];
    for (int b = 0; b < p->N; ++b)
      for (int e = 0; e < 3; ++e) {
        if (e == d) { G[b][e] = dd[b]; continue; }
        int ex = (e == 0), ey = (e == 1), ez = (e == 2);
        G[b][e] = (rd(o, F_PHI_SRC, b, x + ex, y + ey, z + ez) - rd(o, F_PHI_SRC, b, x - ex, y - ey, z - ez) +
                   rd(o, F_PHI_SRC, b, qx + ex, qy + ey, qz + ez) - rd(o, F_PHI_SRC, b, qx - ex, qy - ey, qz - ez)) /
                  (4.0 * p->dx);
      }
    for (int a = 0; a < p->N; ++a) {
      double s = 0.0;
      for (int b = 0; b < p->N; ++b) {
        if (b == a) continue;
        double qv[3], gf[3];
        for (int e = 0; e < 3; ++e) qv[e] = pb[a] * G[b][e] - pb[b] * G[a][e];
        aniso_grad(p, a, b, qv, gf);
        s += p->gamma[a][b] * (-pb[b]) * gf[d];
      }
      j[a] = s;
    }
    return;
  }
  for (int a = 0; a < p->N; ++a) {
    double s = 0.0;
    for (int b = 0; b < p->N; ++b) {
      if (b == a) continue;
      s += p->gamma[a][b] * pb[b] * (pb[b] * dd[a] - pb[a] * dd[b]);
    }
    j[a] = 2.0 * s;
  }
}

/* r_a = delta Psi / delta phi_a at interior cell (x,y,z), C.1 S2 steps 1-5:
 *   r_a = eps (da/dphi_a - div_a) + omega'_a / eps + psi_a h'(phi_a)      */
static void phi_rhs_cell(const pf_oracle* o, int x, int y, int z, double* r) {
  const or_params* p = &o->p;
  const int N = p->N;
  double ph[OR_MAXN], g[OR_MAXN][3], div[OR_MAXN], jp[OR_MAXN], jm[OR_MAXN];
  for (int a = 0; a < N; ++a) { ph[a] = rd(o, F_PHI_SRC, a, x, y, z); div[a] = 0.0; }

  /* 1. divergence of the staggered fluxes (eq. 11) */
  for (int d = 0; d < 3; ++d) {
    phi_face_flux(o, x, y, z, d, jp);                                         /* c+1/2 e_d */
    phi_face_flux(o, x - (d == 0), y - (d == 1), z - (d == 2), d, jm);        /* c-1/2 e_d */
    for (int a = 0; a < N; ++a) div[a] += (jp[a] - jm[a]) / p->dx;
  }
  /* 2. cell-centred gradients, central differences (D3C7) [A10] */
  for (int b = 0; b < N; ++b)
    for (int d = 0; d < 3; ++d) {
      int ex = (d == 0), ey = (d == 1), ez = (d == 2);
      g[b][d] = (rd(o, F_PHI_SRC, b, x + ex, y + ey, z + ez) - rd(o, F_PHI_SRC, b, x - ex, y - ey, z - ez)) /
                (2.0 * p->dx);
    }
  /* mu and T at the cell centre (D3C1 of mu_src, Algorithm 1 line 1) */
  double mu[OR_MAXM];
  for (int i = 0; i < p->M; ++i) mu[i] = rd(o, F_MU_SRC, i, x, y, z);
  double T = temperature(o, (double)z);

  for (int a = 0; a < N; ++a) {
    /* da/dphi_a = 2 sum_{b!=a} gamma_ab (phi_a g_b - phi_b g_a) . g_b  (eq. 4) */
    double dadphi = 0.0;
    if (p->aniso) { /* P2 [B6]: sum_{b!=a} gamma_ab grad_q f(q_ab) . g_b, q_ab = phi_a g_b - phi_b g_a */
      for (int b = 0; b < N; ++b) {
        if (b == a) continue;
        double qv[3], gf[3];
        for (int d = 0; d < 3; ++d) qv[d] = ph[a] * g[b][d] - ph[b] * g[a][d];
        aniso_grad(p, a, b, qv, gf);
        dadphi += p->gamma[a][b] * (gf[0] * g[b][0] + gf[1] * g[b][1] + gf[2] * g[b][2]);
      }
    } else {
    for (int b = 0; b < N; ++b) {
      if (b == a) continue;
      double dot = 0.0;
      for (int d = 0; d < 3; ++d) dot += (ph[a] * g[b][d] - ph[b] * g[a][d]) * g[b][d];
      dadphi += p->gamma[a][b] * dot;
    }
    dadphi *= 2.0;
    }
    /* 3. omega'_a = 16/pi^2 sum_{b!=a} gamma_ab phi_b + sum_{b<d; b,d!=a} gamma_abd phi_b phi_d (eq. 5) */
    double om = 0.0;
    for (int b = 0; b < N; ++b)
      if (b != a) om += p->gamma[a][b] * ph[b];
    om *= 16.0 / (PI_D * PI_D);
    for (int b = 0; b < N; ++b)
      for (int d = b + 1; d < N; ++d)
        if (b != a && d != a) om += gamma3_of(p, a, b, d) * ph[b] * ph[d];
    /* 4. driving force d psi / d phi_a = psi_a(mu,T) h'(phi_a) (eq. 6) */
    double dpsi = psi_of(p, a, mu, T) * dh_of(ph[a]);
    /* 5. */
    r[a] = p->eps * (dadphi - div[a]) + om / p->eps + dpsi;
  }
}

/* ------------------------------------------------------------------------ */
/* Fluctuation term (eq. 7 "+ xi", listing P:L490-495: fluctuation =
 * amplitude * random(-1, 1, kind='philox'); "the counter-based
 * random number generator Philox [31] ... The global cell index and current
 * time step are used as counters/keys").  Reading B4:
 * counter = (x, y, z, step mod 2^32), key = (seed, step / 2^32); the four
 * 32-bit words u_a give U_a = (u_a + 1/2) 2^-31 - 1 in (-1, 1) (exact in
 * fp64) for phases a = 0..N-1.                                              */
/* ------------------------------------------------------------------------ */
static unsigned int mulhilo32(unsigned int a, unsigned int b, unsigned int* hi) {
  const unsigned long long p = (unsigned long long)a * (unsigned long long)b;
  *hi = (unsigned int)(p >> 32);
  return (unsigned int)p;
}

void oracle_philox4x32_10(const unsigned int ctr[4], const unsigned int key[2], unsigned int out[4]) {
  unsigned int c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
  unsigned int k0 = key[0], k1 = key[1];
  for (int round = 0; round < 10; ++round) {
    unsigned int hi0, hi1;
    const unsigned int lo0 = mulhilo32(0xD2511F53u, c0, &hi0);
    const unsigned int lo1 = mulhilo32(0xCD9E8D57u, c2, &hi1);
    const unsigned int n0 = hi1 ^ c1 ^ k0, n1 = lo1, n2 = hi0 ^ c3 ^ k1, n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    k0 += 0x9E3779B9u; /* Weyl sequence key schedule */
    k1 += 0xBB67AE85u;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

void oracle_xi_uniforms(int x, int y, int z, int64_t n, unsigned int seed, double U[4]) {
  const unsigned int ctr[4] = {(unsigned int)x, (unsigned int)y, (unsigned int)z, (unsigned int)(uint64_t)n};
  const unsigned int key[2] = {seed, (unsigned int)((uint64_t)n >> 32)};
  unsigned int u[4];
  oracle_philox4x32_10(ctr, key, u);
  for (int a = 0; a < 4; ++a) U[a] = ((double)u[a] + 0.5) * (1.0 / 2147483648.0) - 1.0;
}

/* C.1 S2 steps 6-8 for one cell: tau, Euler + Lagrange multiplier, projection */
static void phi_update_cell(pf_oracle* o, int x, int y, int z) {
  const or_params* p = &o->p;
  const int N = p->N;
  double r[OR_MAXN], ph[OR_MAXN], xs[OR_MAXN], out[OR_MAXN];
  phi_rhs_cell(o, x, y, z, r);
  for (int a = 0; a < N; ++a) ph[a] = rd(o, F_PHI_SRC, a, x, y, z);
  /* 6. tau = sum_{a<b} tau_ab phi_a phi_b / sum_{a<b} phi_a phi_b [A5] */
  double num = 0.0, den = 0.0, tsum = 0.0;
  int npair = 0;
  for (int a = 0; a < N; ++a)
    for (int b = a + 1; b < N; ++b) {
      num += p->tau[a][b] * ph[a] * ph[b];
      den += ph[a] * ph[b];
      tsum += p->tau[a][b];
      ++npair;
    }
  double tau = den != 0.0 ? num / den : tsum / (double)npair;
  /* 7. tau eps d_t phi_a = -r_a + (1/N) sum_b r_b  (eq. 7 + listing P:L490-495) [A1, A3] */
  double rs = 0.0;
  for (int b = 0; b < N; ++b) rs += r[b];
  double lam = rs / (double)N;
  double f = p->dt / (tau * p->eps);
  /* fluctuation xi_a (eq. 7) [B4]; 0 when off [A17] */
  double xi[OR_MAXN] = {0.0, 0.0, 0.0, 0.0};
  if (p->xi_amp != 0.0) {
    double U[4];
    oracle_xi_uniforms(x, y, z, o->st.step, p->xi_seed, U);
    for (int a = 0; a < N; ++a) xi[a] = p->xi_amp * U[a];
  }
  for (int a = 0; a < N; ++a) xs[a] = ph[a] + f * (-r[a] + lam + xi[a]);
  /* 8. Gibbs-simplex projection [A14, A25] */
  if (p->projection)
    oracle_project_simplex(N, xs, out);
  else
    for (int a = 0; a < N; ++a) out[a] = xs[a];
  for (int a = 0; a < N; ++a) {
    if (g_tr.on) { g_tr.nstore++; continue; }
    o->phi[1 - o->cur][idx(o, a, x, y, z)] = out[a];
  }
}

/* ------------------------------------------------------------------------ */
/* mu-sweep  (Algorithm 1 line 3)                               */
/* ------------------------------------------------------------------------ */

/* Flux F = M grad mu - J_at at the face between p and q = p+e_d (eqs. 8-10,
 * discretised per eq. 11).  All coefficients use phi_src; phi_dst enters only
 * through d_t phi = (phi_dst - phi_src)/dt, for the solids [A8, A11].
 * Tangential derivative = mean of the two adjacent central differences [A9]. */
static void mu_face_flux(const pf_oracle* o, int x, int y, int z, int d, double* F) {
  const or_params* p = &o->p;
  const int N = p->N, M = p->M, L = p->liquid;
  if (g_tr.on && g_tr.virt_flux) {
    for (int i = 0; i < M; ++i) { trace_read(F_FLUX_MU, 4 * i + d, x, y, z); F[i] = 0.0; }
    return;
  }
  int qx = x + (d == 0), qy = y + (d == 1), qz = z + (d == 2);
  double pb[OR_MAXN], gr[OR_MAXN][3], dtp[OR_MAXN];
  for (int a = 0; a < N; ++a) {
    double vp = rd(o, F_PHI_SRC, a, x, y, z), vq = rd(o, F_PHI_SRC, a, qx, qy, qz);
    pb[a] = 0.5 * (vp + vq);
    for (int e = 0; e < 3; ++e) {
      if (e == d) { gr[a][e] = (vq - vp) / p->dx; continue; }
      int ex = (e == 0), ey = (e == 1), ez = (e == 2);
      gr[a][e] = (rd(o, F_PHI_SRC, a, x + ex, y + ey, z + ez) - rd(o, F_PHI_SRC, a, x - ex, y - ey, z - ez) +
                  rd(o, F_PHI_SRC, a, qx + ex, qy + ey, qz + ez) - rd(o, F_PHI_SRC, a, qx - ex, qy - ey, qz - ez)) /
                 (4.0 * p->dx);
    }
    dtp[a] = 0.0;
    if (a != L)
      dtp[a] = ((rd(o, F_PHI_DST, a, x, y, z) - vp) + (rd(o, F_PHI_DST, a, qx, qy, qz) - vq)) / (2.0 * p->dt);
  }
  double mub[OR_MAXM], dmu[OR_MAXM];
  for (int i = 0; i < M; ++i) {
    double vp = rd(o, F_MU_SRC, i, x, y, z), vq = rd(o, F_MU_SRC, i, qx, qy, qz);
    mub[i] = 0.5 * (vp + vq);
    dmu[i] = (vq - vp) / p->dx;
  }
  double Tf = temperature(o, (double)z + (d == 2 ? 0.5 : 0.0));

  /* eq. 9: M = sum_a D_a (dc_a/dmu) g_a(phi)   (D_a left-multiplied) [A7] */
  double Mf[OR_MAXM][OR_MAXM] = {{0}};
  for (int a = 0; a < N; ++a) {
    double chi[OR_MAXM][OR_MAXM];
    chi_of(p, a, Tf, chi);
    for (int i = 0; i < M; ++i)
      for (int j = 0; j < M; ++j) {
        double s = 0.0;
        for (int k = 0; k < M; ++k) s += p->D[a][i][k] * chi[k][j];
        Mf[i][j] += g_of(pb[a]) * s;
      }
  }
  for (int i = 0; i < M; ++i) {
    F[i] = 0.0;
    for (int j = 0; j < M; ++j) F[i] += Mf[i][j] * dmu[j];
  }
  if (!p->antitrapping) return;

  /* eq. 10: J_at = (pi eps/4) sum_{a!=l} g_a h_l / sqrt(phi_a phi_l) d_t phi_a
   *               (n_a . n_l) (c_l - c_a) (x) n_a,   n = grad phi/|grad phi|  [A11] */
  double cl[OR_MAXM];
  conc_of(p, L, mub, Tf, cl);
  double nl2 = 0.0;
  for (int e = 0; e < 3; ++e) nl2 += gr[L][e] * gr[L][e];
  for (int a = 0; a < N; ++a) {
    if (a == L) continue;
    double na2 = 0.0;
    for (int e = 0; e < 3; ++e) na2 += gr[a][e] * gr[a][e];
    /* guards against exact zero (C.6.3) */
    if (!(pb[a] > 0.0 && pb[L] > 0.0 && na2 > 0.0 && nl2 > 0.0)) continue;
    double nrm_a = sqrt(na2), nrm_l = sqrt(nl2);
    double dot = 0.0;
    for (int e = 0; e < 3; ++e) dot += (gr[a][e] / nrm_a) * (gr[L][e] / nrm_l);
    double w = (PI_D * p->eps / 4.0) * g_of(pb[a]) * h_of(pb[L]) / sqrt(pb[a] * pb[L]) * dtp[a] * dot;
    double ca[OR_MAXM];
    conc_of(p, a, mub, Tf, ca);
    for (int i = 0; i < M; ++i) F[i] -= w * (cl[i] - ca[i]) * (gr[a][d] / nrm_a);
  }
}

/* C.1 S4 for one cell: mu' = mu + dt chi^{-1} (div - S - Q)   (eq. 8) */
static void mu_update_cell(pf_oracle* o, int x, int y, int z) {
  const or_params* p = &o->p;
  const int N = p->N, M = p->M;
  double div[OR_MAXM] = {0}, Fp[OR_MAXM], Fm[OR_MAXM];
  for (int d = 0; d < 3; ++d) {
    mu_face_flux(o, x, y, z, d, Fp);
    mu_face_flux(o, x - (d == 0), y - (d == 1), z - (d == 2), d, Fm);
    for (int i = 0; i < M; ++i) div[i] += (Fp[i] - Fm[i]) / p->dx;
  }
  double mu[OR_MAXM], ph[OR_MAXN], phn[OR_MAXN];
  for (int i = 0; i < M; ++i) mu[i] = rd(o, F_MU_SRC, i, x, y, z);
  for (int a = 0; a < N; ++a) { ph[a] = rd(o, F_PHI_SRC, a, x, y, z); phn[a] = rd(o, F_PHI_DST, a, x, y, z); }
  double T = temperature(o, (double)z);
  double dTdt = -p->G * p->v; /* d_t T of T0 + G(z - v t) */

  /* chi = dc/dmu = sum_a h_a chi_a;  S = sum_a c_a h'_a d_t phi_a;  Q = sum_a h_a dc_a/dT d_t T */
  double chi[OR_MAXM][OR_MAXM] = {{0}}, S[OR_MAXM] = {0}, Q[OR_MAXM] = {0};
  for (int a = 0; a < N; ++a) {
    double ch[OR_MAXM][OR_MAXM], c[OR_MAXM], cT[OR_MAXM];
    chi_of(p, a, T, ch);
    conc_of(p, a, mu, T, c);
    dcdT_of(p, a, mu, cT);
    double h = h_of(ph[a]), dh = dh_of(ph[a]);
    double dtphi = (phn[a] - ph[a]) / p->dt; /* [A12] */
    for (int i = 0; i < M; ++i) {
      for (int j = 0; j < M; ++j) chi[i][j] += h * ch[i][j];
      S[i] += c[i] * dh * dtphi;
      Q[i] += h * cT[i] * dTdt;
    }
  }
  double rhs[OR_MAXM], upd[OR_MAXM];
  for (int i = 0; i < M; ++i) rhs[i] = div[i] - S[i] - Q[i];
  if (M == 1) {
    upd[0] = rhs[0] / chi[0][0];
  } else { /* closed-form 2x2 inverse (C.6.5) */
    double det = chi[0][0] * chi[1][1] - chi[0][1] * chi[1][0];
    upd[0] = (chi[1][1] * rhs[0] - chi[0][1] * rhs[1]) / det;
    upd[1] = (-chi[1][0] * rhs[0] + chi[0][0] * rhs[1]) / det;
  }
  for (int i = 0; i < M; ++i) {
    if (g_tr.on) { g_tr.nstore++; continue; }
    o->mu[1 - o->cur][idx(o, i, x, y, z)] = mu[i] + p->dt * upd[i];
  }
}

/* ------------------------------------------------------------------------ */
/* Ghost layers: "communication and boundary handling" (Alg. 1 lines 2, 4)   */
/* Ordered x -> y -> z so that edges and corners are consistent [A15, C.6.6] */
/* ------------------------------------------------------------------------ */
static void fill_ghosts(pf_oracle* o, double* f, int ncomp, int is_mu) {
  const int n[3] = {o->g.nx, o->g.ny, o->g.nz};
  for (int d = 0; d < 3; ++d) {
    /* ranges of the other two axes: interior for axes after d, full for axes before d */
    int lo[3], hi[3];
    for (int e = 0; e < 3; ++e) {
      lo[e] = e < d ? -1 : 0;
      hi[e] = e < d ? n[e] : n[e] - 1;
    }
    for (int c = 0; c < ncomp; ++c)
      for (int side = 0; side < 2; ++side) {
        int bc = side ? o->g.bc_hi[d] : o->g.bc_lo[d];
        int gpos = side ? n[d] : -1;                     /* ghost index */
        int src_per = side ? 0 : n[d] - 1;               /* periodic image */
        int src_neu = side ? n[d] - 1 : 0;               /* adjacent interior */
        int a0 = (d == 0) ? 1 : 0, a1 = (d == 2) ? 1 : 2; /* the two other axes */
        for (int u = lo[a0]; u <= hi[a0]; ++u)
          for (int w = lo[a1]; w <= hi[a1]; ++w) {
            int gi[3], si[3];
            gi[d] = gpos; gi[a0] = u; gi[a1] = w;
            si[a0] = u; si[a1] = w;
            double val;
            if (bc == OR_BC_PERIODIC) {
              si[d] = src_per;
              val = f[idx(o, c, si[0], si[1], si[2])];
            } else if (bc == OR_BC_DIRICHLET_MU && is_mu) {
              val = o->p.mu_inf[c];
            } else {
              si[d] = src_neu;
              val = f[idx(o, c, si[0], si[1], si[2])];
            }
            f[idx(o, c, gi[0], gi[1], gi[2])] = val;
          }
      }
  }
}

/* ------------------------------------------------------------------------ */
/* Moving window (S6) [A16]                                                  */
/* ------------------------------------------------------------------------ */
int oracle_front_height(const pf_oracle* o) {
  int H = -1;
  const int L = o->p.liquid;
  for (int z = 0; z < o->g.nz; ++z)
    for (int y = 0; y < o->g.ny; ++y)
      for (int x = 0; x < o->g.nx; ++x)
        if (o->phi[o->cur][idx(o, L, x, y, z)] < 0.5 && z > H) H = z;
  return H;
}

int oracle_shift_window(pf_oracle* o, int k) {
  if (k < 0 || k > o->g.nz) return -1;
  if (k == 0) return 0;
  const int nz = o->g.nz;
  double* ph = o->phi[o->cur];
  double* mu = o->mu[o->cur];
  for (int z = 0; z < nz; ++z)
    for (int y = 0; y < o->g.ny; ++y)
      for (int x = 0; x < o->g.nx; ++x) {
        for (int a = 0; a < o->p.N; ++a)
          ph[idx(o, a, x, y, z)] = z + k < nz ? ph[idx(o, a, x, y, z + k)] : (a == o->p.liquid ? 1.0 : 0.0);
        for (int i = 0; i < o->p.M; ++i)
          mu[idx(o, i, x, y, z)] = z + k < nz ? mu[idx(o, i, x, y, z + k)] : o->p.mu_inf[i];
      }
  o->st.z_off += k;
  fill_ghosts(o, ph, o->p.N, 0);
  fill_ghosts(o, mu, o->p.M, 1);
  return 0;
}

static void window_check(pf_oracle* o) {
  if (o->p.window_check <= 0 || o->st.step % o->p.window_check != 0) return;
  int H = oracle_front_height(o);
  int thr = (int)floor(o->p.window_frac * (double)o->g.nz);
  if (H > thr) oracle_shift_window(o, H - thr);
}

/* ------------------------------------------------------------------------ */
/* Driver                                                                    */
/* ------------------------------------------------------------------------ */
pf_oracle* oracle_create(const or_grid* g, const or_params* p) {
  if (p->N < 2 || p->N > OR_MAXN || p->M < 1 || p->M > OR_MAXM || p->liquid < 0 || p->liquid >= p->N) return NULL;
  if (g->nx < 1 || g->ny < 1 || g->nz < 1) return NULL;
  pf_oracle* o = (pf_oracle*)calloc(1, sizeof *o);
  if (!o) return NULL;
  o->g = *g;
  o->p = *p;
  o->sx = g->nx + 2; o->sy = g->ny + 2; o->sz = g->nz + 2;
  size_t cells = (size_t)o->sx * o->sy * o->sz;
  for (int l = 0; l < 2; ++l) {
    o->phi[l] = (double*)calloc(cells * p->N, sizeof(double));
    o->mu[l] = (double*)calloc(cells * p->M, sizeof(double));
  }
  return o;
}

void oracle_destroy(pf_oracle* o) {
  if (!o) return;
  for (int l = 0; l < 2; ++l) { free(o->phi[l]); free(o->mu[l]); }
  free(o);
}

int oracle_init(pf_oracle* o, const double* phi, const double* mu) {
  const int nx = o->g.nx, ny = o->g.ny, nz = o->g.nz;
  o->cur = 0;
  for (int a = 0; a < o->p.N; ++a)
    for (int z = 0; z < nz; ++z)
      for (int y = 0; y < ny; ++y)
        for (int x = 0; x < nx; ++x)
          o->phi[0][idx(o, a, x, y, z)] = phi[(((size_t)a * nz + z) * ny + y) * nx + x];
  for (int i = 0; i < o->p.M; ++i)
    for (int z = 0; z < nz; ++z)
      for (int y = 0; y < ny; ++y)
        for (int x = 0; x < nx; ++x)
          o->mu[0][idx(o, i, x, y, z)] = mu[(((size_t)i * nz + z) * ny + y) * nx + x];
  o->st.step = 0;
  o->st.z_off = 0;
  fill_ghosts(o, o->phi[0], o->p.N, 0);
  fill_ghosts(o, o->mu[0], o->p.M, 1);
  return 0;
}

int oracle_download(const pf_oracle* o, double* phi, double* mu) {
  const int nx = o->g.nx, ny = o->g.ny, nz = o->g.nz;
  for (int a = 0; a < o->p.N; ++a)
    for (int z = 0; z < nz; ++z)
      for (int y = 0; y < ny; ++y)
        for (int x = 0; x < nx; ++x)
          phi[(((size_t)a * nz + z) * ny + y) * nx + x] = o->phi[o->cur][idx(o, a, x, y, z)];
  for (int i = 0; i < o->p.M; ++i)
    for (int z = 0; z < nz; ++z)
      for (int y = 0; y < ny; ++y)
        for (int x = 0; x < nx; ++x)
          mu[(((size_t)i * nz + z) * ny + y) * nx + x] = o->mu[o->cur][idx(o, i, x, y, z)];
  return 0;
}

void oracle_get_state(const pf_oracle* o, or_state* s) { *s = o->st; }
void oracle_set_state(pf_oracle* o, const or_state* s) { o->st = *s; }

static void phi_sweep(pf_oracle* o) {
  const int nx = o->g.nx, ny = o->g.ny, nz = o->g.nz;
#ifdef _OPENMP
#pragma omp parallel for schedule(static) num_threads(g_threads > 0 ? g_threads : 1) if (g_threads > 0)
#endif
  for (int z = 0; z < nz; ++z)
    for (int y = 0; y < ny; ++y)
      for (int x = 0; x < nx; ++x) phi_update_cell(o, x, y, z);
}

static void mu_sweep(pf_oracle* o) {
  const int nx = o->g.nx, ny = o->g.ny, nz = o->g.nz;
#ifdef _OPENMP
#pragma omp parallel for schedule(static) num_threads(g_threads > 0 ? g_threads : 1) if (g_threads > 0)
#endif
  for (int z = 0; z < nz; ++z)
    for (int y = 0; y < ny; ++y)
      for (int x = 0; x < nx; ++x) mu_update_cell(o, x, y, z);
}

/* One time step = Algorithm 1 + window check (S6) */
int oracle_step(pf_oracle* o, int64_t nsteps) {
  for (int64_t n = 0; n < nsteps; ++n) {
    phi_sweep(o);                                 /* line 1 */
    fill_ghosts(o, o->phi[1 - o->cur], o->p.N, 0); /* line 2 */
    mu_sweep(o);                                  /* line 3 */
    fill_ghosts(o, o->mu[1 - o->cur], o->p.M, 1);  /* line 4 */
    o->cur = 1 - o->cur;                          /* line 5 */
    o->st.step += 1;
    window_check(o);
  }
  return 0;
}

/* phi-sweep only (C.7 split diagnosis): phi_dst from phi_src, mu unchanged */
int oracle_step_phi_only(pf_oracle* o) {
  phi_sweep(o);
  fill_ghosts(o, o->phi[1 - o->cur], o->p.N, 0);
  /* carry mu over unchanged so that the swapped state is complete */
  size_t cells = (size_t)o->sx * o->sy * o->sz;
  memcpy(o->mu[1 - o->cur], o->mu[o->cur], cells * o->p.M * sizeof(double));
  o->cur = 1 - o->cur;
  o->st.step += 1;
  return 0;
}

int oracle_phi_rhs(pf_oracle* o, double* r) {
  const int nx = o->g.nx, ny = o->g.ny, nz = o->g.nz, N = o->p.N;
  for (int z = 0; z < nz; ++z)
    for (int y = 0; y < ny; ++y)
      for (int x = 0; x < nx; ++x) {
        double rc[OR_MAXN];
        phi_rhs_cell(o, x, y, z, rc);
        for (int a = 0; a < N; ++a) r[(((size_t)a * nz + z) * ny + y) * nx + x] = rc[a];
      }
  return 0;
}

/* Pin P14: trace the loads of one cell update and count distinct values */
int oracle_footprint(pf_oracle* o, int which, int x, int y, int z, int* stores) {
  memset(&g_tr, 0, sizeof g_tr);
  g_tr.cx = x; g_tr.cy = y; g_tr.cz = z;
  g_tr.on = 1;
  switch (which) {
    case 0: phi_update_cell(o, x, y, z); break; /* phi-full */
    case 1: {                                   /* phi-flux: the 3 lower faces */
      double j[OR_MAXN];
      for (int d = 0; d < 3; ++d) {
        phi_face_flux(o, x - (d == 0), y - (d == 1), z - (d == 2), d, j);
        g_tr.nstore += o->p.N;
      }
      break;
    }
    case 2: g_tr.virt_flux = 1; phi_update_cell(o, x, y, z); break; /* phi-cell */
    case 3: mu_update_cell(o, x, y, z); break;                      /* mu-full */
    case 4: {                                                       /* mu-flux */
      double F[OR_MAXM];
      for (int d = 0; d < 3; ++d) {
        mu_face_flux(o, x - (d == 0), y - (d == 1), z - (d == 2), d, F);
        g_tr.nstore += o->p.M;
      }
      break;
    }
    case 5: g_tr.virt_flux = 1; mu_update_cell(o, x, y, z); break; /* mu-cell */
    default: g_tr.on = 0; return -1;
  }
  int n = g_tr.n;
  if (stores) *stores = g_tr.nstore;
  memset(&g_tr, 0, sizeof g_tr);
  return n;
}
