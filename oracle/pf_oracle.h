/*
 * pf_oracle.h -- CPU ORACLE for the grand-potential multiphase-field time step
 * of Bauer et al., "Code Generation for Massively Parallel Phase-Field
 * Simulations" (SC'19).  Citations "P:Lx-y" are lines of the paper text
 * (/root/reference/PAPER.md); "A<n>" are the readings of DESIGN.md §3.
 *
 * THIS IS TEST INFRASTRUCTURE.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load it.  It shares no
 * code, header, table or constant with the CUDA path
 * (paper_conf_sc_0003hehshhkwnr19_b200/csrc), and never imports it.
 *
 * Plain, slow, obviously-correct fp64: generic N (2..4 phases) and
 * M = K-1 (1..2 chemical potentials), any liquid index, one ghost layer.
 */
#ifndef PF_ORACLE_H
#define PF_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define OR_MAXN 4
#define OR_MAXM 2

/* boundary kinds per side (reading A15) */
#define OR_BC_PERIODIC 0
#define OR_BC_NEUMANN 1      /* phi and mu: ghost = adjacent interior value   */
#define OR_BC_DIRICHLET_MU 2 /* phi Neumann, mu ghost = mu_inf              */

typedef struct {
  int N;      /* phases                                   P:L382-388 (eq. 4) */
  int M;      /* chemical potentials, K-1                 P:L426 (eq. 6)     */
  int liquid; /* index l of the liquid phase              P:L563 (eq. 10)    */
  double dx, dt, eps;
  double gamma[OR_MAXN][OR_MAXN];           /* gamma_ab  eq. 4/5           */
  double gamma3[OR_MAXN][OR_MAXN][OR_MAXN]; /* gamma_abd eq. 5             */
  double tau[OR_MAXN][OR_MAXN];             /* tau_ab        */
  double A0[OR_MAXN][OR_MAXM][OR_MAXM], A1[OR_MAXN][OR_MAXM][OR_MAXM];
  double B0[OR_MAXN][OR_MAXM], B1[OR_MAXN][OR_MAXM];
  double C0[OR_MAXN], C1[OR_MAXN];          /* eq. 6, affine in T          */
  double D[OR_MAXN][OR_MAXM][OR_MAXM];      /* D_alpha, eq. 9              */
  double T0, G, v;                          /* frozen T (reading A13)      */
  double mu_inf[OR_MAXM];                   /* inflow / Dirichlet value    */
  double window_frac;                       /* moving window (A16)         */
  int window_check;                         /* 0 = window off              */
  /* debug switches */
  int antitrapping; /* 1 = eq. 10 on (default), 0 = off                    */
  int projection;   /* 1 = Gibbs-simplex projection on (default), 0 = off  */
  /* fluctuation term xi of eq. 7, reading B4:
   * xi_a = xi_amp * U_a, U_a uniform in (-1, 1) from Philox4x32-10 keyed by
   * the global cell index and the time step; 0 = off (reading A17)        */
  double xi_amp;
  unsigned int xi_seed;
  /* P2 parameterisation: anisotropic
   * gradient energy a = sum_{a<b} gamma_ab A_ab(R_ab q_ab)^2 |q_ab|^2 (eq. 4,
   * P:L382-398), reading B6: cubic A_ab(p) = 1 - delta_ab (3 - 4 sum_i p_i^4
   * / |p|^4), R_ab orthonormal, both symmetric in (a, b).  The face flux of
   * eq. 11 then needs the whole face gradient (normal + mean tangential
   * central differences, as for mu [A9]): a 19-point phi stencil.
   * aniso = 0: A = 1 (P1, 7-point phi stencil).                          */
  int aniso;
  double aniso_delta[OR_MAXN][OR_MAXN];
  double aniso_R[OR_MAXN][OR_MAXN][3][3];
} or_params;

typedef struct {
  int nx, ny, nz;
  int bc_lo[3], bc_hi[3]; /* OR_BC_* for x, y, z */
} or_grid;

typedef struct or_state_s {
  int64_t step;  /* completed steps; t_n = step * dt */
  int64_t z_off; /* window offset, in cells          */
} or_state;

typedef struct pf_oracle pf_oracle;

pf_oracle* oracle_create(const or_grid* g, const or_params* p);
void oracle_destroy(pf_oracle* o);
/* interior-only SoA arrays: phi[N][nz][ny][nx], mu[M][nz][ny][nx] */
int oracle_init(pf_oracle* o, const double* phi, const double* mu);
int oracle_step(pf_oracle* o, int64_t nsteps);
int oracle_step_phi_only(pf_oracle* o); /* C.7 split diagnosis          */
int oracle_shift_window(pf_oracle* o, int k);
int oracle_download(const pf_oracle* o, double* phi, double* mu);
void oracle_get_state(const pf_oracle* o, or_state* s);
void oracle_set_state(pf_oracle* o, const or_state* s);
void oracle_set_threads(int n); /* OpenMP threads for timing only; 0 = serial */

/* debug / pin hooks */
/* r_alpha = delta Psi / delta phi_alpha on every interior cell (C.1 S2.5) */
int oracle_phi_rhs(pf_oracle* o, double* r);
/* Euclidean projection onto the Gibbs simplex (reading A14)               */
void oracle_project_simplex(int N, const double* x, double* out);
/* Philox4x32-10 (Salmon et al., SC'11), the counter-based RNG of P:L669-676:
 * out = the 10-round bijection of counter ctr under key key.               */
void oracle_philox4x32_10(const unsigned int ctr[4], const unsigned int key[2], unsigned int out[4]);
/* The four uniforms U in (-1, 1) of cell (x, y, z) at step n (reading B4). */
void oracle_xi_uniforms(int x, int y, int z, int64_t n, unsigned int seed, double U[4]);
/* front height H of S6 (-1 if no solid cell) */
int oracle_front_height(const pf_oracle* o);
/* Table-1 footprint (pin P14): which = 0 phi-full, 1 phi-flux, 2 phi-cell,
 * 3 mu-full, 4 mu-flux, 5 mu-cell.  Returns #distinct loaded values,
 * *stores = #values stored.  Traces one interior cell (x,y,z). */
int oracle_footprint(pf_oracle* o, int which, int x, int y, int z, int* stores);

#ifdef __cplusplus
}
#endif
#endif
