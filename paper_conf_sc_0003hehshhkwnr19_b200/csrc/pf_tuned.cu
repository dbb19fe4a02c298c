// pf_tuned.cu -- generic (ahead-of-time) instantiation of the tuned sweeps
// of pf_sweeps.cuh: parameters in the kernel-parameter constant bank,
// geometry at run time.  The specialised build (pf_jit.cu) compiles the same
// bodies with both folded in.
#include "pf_internal.h"
// the generic (run-time parameter) build has less register headroom than the
// specialised one: no register prefetch of the next plane and no unrolled
// phi loop (both spill here)
#define PF_MU_RPF 0
#define PF_PHI_UNROLL 1
#include "pf_sweeps.cuh"

namespace pf {

// dispatch on the liquid index (compile-time L) and the T-dependence of A (TA)
#define PF_DISPATCH_TA(TA, ...)                  \
  if (TA) {                                      \
    constexpr bool TT = true;                    \
    __VA_ARGS__;                                 \
  } else {                                       \
    constexpr bool TT = false;                   \
    __VA_ARGS__;                                 \
  }
#define PF_DISPATCH(L, TA, ...)                                        \
  switch (L) {                                                         \
    case 0: { constexpr int LL = 0; PF_DISPATCH_TA(TA, __VA_ARGS__); } break; \
    case 1: { constexpr int LL = 1; PF_DISPATCH_TA(TA, __VA_ARGS__); } break; \
    case 2: { constexpr int LL = 2; PF_DISPATCH_TA(TA, __VA_ARGS__); } break; \
    default: { constexpr int LL = 3; PF_DISPATCH_TA(TA, __VA_ARGS__); } break; \
  }


template <int L, bool TA>
__global__ void __launch_bounds__(TX* TY, 2) k_phi_tuned(DevParams P, Geom g, const double* __restrict__ ps,
                                                         const double* __restrict__ ms, double* __restrict__ pd) {
  phi_tuned_body<DevParams, Geom, L, TA>(P, P, g, ps, ms, pd);
}

template <int L, bool TA>
__global__ void __launch_bounds__(TX* MU_TY, MU_TY == 4 ? 3 : 16 / MU_TY) k_mu_tuned(DevParams P, Geom g, TileSel ts,
                                                                  const double* __restrict__ ps,
                                                                  const double* __restrict__ pd,
                                                                  const double* __restrict__ ms,
                                                                  double* __restrict__ md) {
  mu_tuned_body<DevParams, Geom, L, TA, MU_TY>(P, P, g, ts, ps, pd, ms, md);
}

dim3 tuned_block() { return dim3(TX, TY); }
dim3 tuned_block_phi(int pty) { return dim3(TX, pty); }
dim3 tuned_block_mu(int mty, int mtx) { return dim3(mtx, mty); }
dim3 tuned_grid_phi(const Geom& g, int pty, int zc, int txc) {
  if (zc <= 0) zc = ZC_PHI;
  return dim3((g.nx + txc - 1) / txc, (g.ny + pty - 1) / pty, (g.nz + zc - 1) / zc);
}
dim3 tuned_grid_mu(const Geom& g, int mty, int zc, int mtx) {
  if (zc <= 0) zc = ZC_MU;
  return dim3((g.nx + mtx - 1) / mtx, (g.ny + mty - 1) / mty, (g.nz + zc - 1) / zc);
}
size_t tuned_mu_smem(int mty, int mtx) {
  return (size_t)(D_NV * (mtx + 2) * (mty + 2) + M * mty * (mtx + 1) + M * (mty + 1) * mtx) * sizeof(double);
}
int tuned_mu_ty_default() { return MU_TY; }

size_t tuned_phi_smem() { return 0; }  // static shared memory only

template <int L, bool TA>
static void phi_launch(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                       cudaStream_t s) {
  Geom g0 = g;
  g0.xwrap = 0;  // the generic build leaves the x ghost columns to the ghost fill
  k_phi_tuned<L, TA><<<tuned_grid_phi(g0, TY, 0), tuned_block(), 0, s>>>(P, g0, ps, ms, pd);
}

void launch_phi_tuned(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                      cudaStream_t s) {
  PF_DISPATCH(P.liquid, P.TA, (phi_launch<LL, TT>(P, g, ps, ms, pd, s)));
}


template <int L, bool TA>
static void mu_launch(const DevParams& P, const Geom& g, const TileSel& ts, dim3 grid, const double* ps,
                      const double* pd, const double* ms, double* md, cudaStream_t s) {
  static bool attr = false;  // per instantiation
  if (!attr) {
    cudaFuncSetAttribute(k_mu_tuned<L, TA>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tuned_mu_smem(MU_TY));
    attr = true;
  }
  k_mu_tuned<L, TA><<<grid, tuned_block_mu(MU_TY), tuned_mu_smem(MU_TY), s>>>(P, g, ts, ps, pd, ms, md);
}

void launch_mu_tuned(const DevParams& P, const Geom& g, const TileSel* ts, dim3 grid, const double* ps,
                     const double* pd, const double* ms, double* md, cudaStream_t s) {
  TileSel all = {{0, 0, 0}, {0, 0, 0}, {0, 0, 0}, 0};
  const TileSel& t = ts ? *ts : all;
  const dim3 gr = ts ? grid : tuned_grid_mu(g, MU_TY, 0);
  PF_DISPATCH(P.liquid, P.TA, (mu_launch<LL, TT>(P, g, t, gr, ps, pd, ms, md, s)));
}


}  // namespace pf
