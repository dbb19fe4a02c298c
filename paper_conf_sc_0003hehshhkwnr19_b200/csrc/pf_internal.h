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

// Geometry of one block in the padded ghosted layout (pf_layout): one ghost
// layer (indices -1 and n) inside an allocated guard ring of width 2 in y and
// z (and >= 2 in x), so that kernels may read any index in [-2, n+1] without
// bounds checks (edge threads of ragged tiles clamp to the ghost cell).
constexpr int GUARD = 2;
struct Geom {
  int nx, ny, nz;
  int z0;  // global z index of local interior plane 0
  int64_t pitch, plane, field, xoff;
  // cell (x,y,z), each in [-2, n+1] -> linear index
  __host__ __device__ __forceinline__ int64_t at(int x, int y, int z) const {
    return (int64_t)(z + GUARD) * plane + (int64_t)(y + GUARD) * pitch + xoff + x;
  }
};

// Scalars and coefficients of the model, passed by value to every kernel
// (kernel-parameter constant bank: DFMA constant operands, no loads), so that
// several contexts may coexist in one process.  T-dependent coefficients are
// stored as value = c0 + T c1 (eq. 6: A, B, C affine in T).
struct DevParams {
  double dx, dt, eps;
  double inv_dt;
  double inv_dx2;       // 1 / dx^2
  double phi_grad_c;    // eps / dx^2
  double inv_eps;
  double dt_over_eps;
  double at_c;          // dx * pi eps / (8 dt): anti-trapping prefactor in unscaled units
  double dTdt;          // -G v
  double Tbase, Tdz;    // T(local plane k) = Tbase + Tdz k  (set per step)  [A13]
  double mu_inf[M];
  // phi-sweep
  double g[N][N];       // gamma_ab (diag 0)
  double og[N][N];      // 16/pi^2 gamma_ab
  double g3[N][3];      // gamma_abd for the 3 pairs (b<d, b,d != a) of phase a, see kOtherPair()
  double tau[6];        // tau_ab for pairs (0,1),(0,2),(0,3),(1,2),(1,3),(2,3)
  double inv_tau_mean;  // 1 / mean tau_ab (tau of a pure cell, reading A5)
  double psiA[N][3], psiA1[N][3];  // mu.A mu = a00 m0^2 + (a01+a10) m0 m1 + a11 m1^2
  double B0[N][M], B1[N][M];
  double C0[N], C1[N];
  // mu-sweep
  double chi0[N][3], chi1[N][3];   // chi_a = dc_a/dmu = -(A + A^T) (sym: 00, 01, 11)  [A6]
  double P0[N][4], P1[N][4];       // D_a chi_a (row-major 00 01 10 11), eq. 9  [A7]
  double dchi0[NSOL][3], dchi1[NSOL][3];  // chi_l - chi_s
  double dB0[NSOL][M], dB1[NSOL][M];      // B_l - B_s
  double dcT[N][5];     // dc_a/dT = -(A1 + A1^T) mu - B1: [s00, s01, s11, -B1_0, -B1_1]
  int liquid;
  int TA;               // A1 != 0: chi and the mobility depend on T
};

// ---- launchers (defined in the kernel TUs) ------------------------------
void launch_phi_naive(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                      cudaStream_t s);
void launch_mu_naive(const DevParams& P, const Geom& g, const double* ps, const double* pd, const double* ms,
                     double* md, cudaStream_t s);
void launch_phi_tuned(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                      cudaStream_t s);
void launch_mu_tuned(const DevParams& P, const Geom& g, const double* ps, const double* pd, const double* ms,
                     double* md, cudaStream_t s);
void launch_ghost_stage(const Geom& g, int d, int klo, int khi, double* f, int ncomp, const double* dirichlet,
                        cudaStream_t s);
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
