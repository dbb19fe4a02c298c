// pf_internal.h -- internal types of the B200 phase-field library (not ABI).
//
// Shared by the host runtime (pf_api.cu) and the kernels (pf_*.cu).  Nothing
// here is shared with the oracle (oracle/), by construction.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/pf.h"

namespace pf {

constexpr int N = PF_N;
constexpr int M = PF_M;
constexpr int NSOL = N - 1;

// Per-plane coefficient table (step a1: frozen T hoisted out of the cell
// loops, P:L700-708 / P:L1185-1193).  One row per interior z-plane k for
// cell-centred quantities at T(k), one row per plane for x/y faces (T(k)),
// one row per z-face k-1/2 .. nz-1/2 (T(k+1/2)).  Rows are padded to 16 B.
// cell row: psi coefficients, chi_a = dc_a/dmu (sym), B_a
constexpr int TC_PSI = 0;              // [N][6] a00, 2 a01, a11, b0, b1, c
constexpr int TC_CHI = TC_PSI + N * 6; // [N][3] chi00, chi01, chi11
constexpr int TC_B = TC_CHI + N * 3;   // [N][2]
constexpr int TC_SIZE = TC_B + N * 2;  // 44
// face row: P_a = D_a chi_a (mobility, eq. 9), solid s: dchi = chi_l - chi_s (sym), dB = B_l - B_s
constexpr int TF_P = 0;                   // [N][4] p00 p01 p10 p11
constexpr int TF_DCHI = TF_P + N * 4;     // [NSOL][3]
constexpr int TF_DB = TF_DCHI + NSOL * 3; // [NSOL][2]
constexpr int TF_SIZE = TF_DB + NSOL * 2; // 31
constexpr int TF_STRIDE = 32;

// Geometry of one block in the padded ghosted layout (pf_layout).
struct Geom {
  int nx, ny, nz;
  int z0;  // global z index of local interior plane 0
  int64_t pitch, plane, field, xoff;
  // interior cell (x,y,z) -> linear index
  __host__ __device__ __forceinline__ int64_t at(int x, int y, int z) const {
    return (int64_t)(z + 1) * plane + (int64_t)(y + 1) * pitch + xoff + x;
  }
};

// Scalars of the model, passed by value to every kernel (kernel-parameter
// constant bank), so that several contexts may coexist in one process.
struct DevParams {
  double dx, dt, eps;
  double inv_dt;
  double inv_dx2;       // 1 / dx^2
  double phi_grad_c;    // eps / dx^2
  double inv_eps;
  double dt_over_eps;
  double g[N][N];       // gamma_ab (diag 0)
  double og[N][N];      // 16/pi^2 gamma_ab
  double g3[N][3];      // gamma_abd for the 3 pairs (b<d, b,d != a) of phase a, see pair_of()
  double tau[6];        // tau_ab for pairs (0,1),(0,2),(0,3),(1,2),(1,3),(2,3)
  double tau_mean;
  double dcT[N][5];     // dc_a/dT = -(A1 + A1^T) mu - B1: [s00, s01, s11, -B1_0, -B1_1]
  double dTdt;          // -G v
  double at_c;          // dx * pi eps / (8 dt): anti-trapping prefactor in unscaled units
  double mu_inf[M];
  double T0, G, v;
  int liquid;
};

// Kernel-side table pointers for the current step.
struct Tables {
  const double* cell;  // [nz][TC_SIZE]
  const double* fxy;   // [nz][TF_STRIDE]
  const double* fz;    // [nz+1][TF_STRIDE], row k+1 = face k+1/2
};

// ---- launchers (defined in the kernel TUs) ------------------------------
size_t table_doubles(int nz);  // TC_SIZE % 2 == 0 and TF_STRIDE = 32 keep rows 16-B aligned
Tables table_view(const double* tab, int nz);
void launch_tables(const pf_params& p, int liquid, const Geom& g, double t, int64_t z_off, double* tab, cudaStream_t s);
void launch_phi_naive(const DevParams& P, const Geom& g, const Tables& T, const double* ps, const double* ms,
                      double* pd, cudaStream_t s);
void launch_mu_naive(const DevParams& P, const Geom& g, const Tables& T, const double* ps, const double* pd,
                     const double* ms, double* md, cudaStream_t s);
void launch_phi_sweep(int variant, const DevParams& P, const Geom& g, const Tables& T, const double* phi_src,
                      const double* mu_src, double* phi_dst, cudaStream_t s);
void launch_mu_sweep(int variant, const DevParams& P, const Geom& g, const Tables& T, const double* phi_src,
                     const double* phi_dst, const double* mu_src, double* mu_dst, cudaStream_t s);
// ghost fill of ncomp components for the sides whose `local[side]` flag is set
// (periodic wrap within this block, Neumann, Dirichlet); sides handled by a
// halo exchange are skipped.
struct BCSpec {
  int kind_lo[3], kind_hi[3];  // PF_BC_* ; -1 = filled by exchange
};
void launch_ghost_fill(const Geom& g, const BCSpec& bc, double* f, int ncomp, const double* dirichlet, cudaStream_t s);
void launch_shift(const Geom& g, int k, int liquid, const double* mu_inf, const double* phi_src, const double* mu_src,
                  double* phi_dst, double* mu_dst, cudaStream_t s);
void launch_front_height(const Geom& g, int liquid, const double* phi, int* out, cudaStream_t s);
void launch_monitor(const Geom& g, const double* phi, unsigned long long* out2, cudaStream_t s);
void launch_copy_interior(const Geom& g, int ncomp, const double* src, double* dst, int to_packed, cudaStream_t s);
void launch_check_fields(const Geom& g, const double* phi, unsigned long long* out2, cudaStream_t s);
// face pack/unpack for halo exchange along dimension d (0..2): the slab at
// interior index `plane_idx` (send) or ghost index (recv), extended ranges
// for the dimensions before d (so edges travel with the x->y->z ordering).
size_t halo_slab_elems(const Geom& g, int d);
void launch_pack(const Geom& g, int d, int src_idx, int ncomp, const double* f, double* buf, cudaStream_t s);
void launch_unpack(const Geom& g, int d, int dst_idx, int ncomp, double* f, const double* buf, cudaStream_t s);

}  // namespace pf
