// pf_kernels.cu -- coefficient tables, the straightforward ("naive") sweeps,
// ghost layers, moving window, reductions and field copies.
//
// The naive sweeps map one thread to one cell and compute every face flux
// twice (the paper's "full" kernels).  They are the parity
// baseline and the ncu reference for the tuned z-marching kernels
// (pf_tuned.cu).
#include <math.h>

#include "pf_internal.h"
#include "pf_model.cuh"

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



// ---------------------------------------------------------------------------
// Naive phi-sweep: one thread per cell, 6 faces each (Algorithm 1 line 1).
// ---------------------------------------------------------------------------
template <int L, bool TA>
__global__ void __launch_bounds__(256) k_phi_naive(DevParams P, Geom g, const double* __restrict__ ps,
                                                   const double* __restrict__ ms, double* __restrict__ pd) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const int64_t c = g.at(x, y, z);
  const int64_t F = g.field;
  double ph[N], gd[N][3], divh[N] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll
  for (int a = 0; a < N; ++a) ph[a] = __ldg(ps + a * F + c);
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    const int64_t st = d == 0 ? 1 : (d == 1 ? g.pitch : g.plane);
    double fm[N], fpl[N], jp[N], jm[N];
#pragma unroll
    for (int a = 0; a < N; ++a) {
      fm[a] = __ldg(ps + a * F + c - st);
      fpl[a] = __ldg(ps + a * F + c + st);
      gd[a][d] = fpl[a] - fm[a];
    }
    phi_face(P, ph, fpl, jp);
    phi_face(P, fm, ph, jm);
#pragma unroll
    for (int a = 0; a < N; ++a) divh[a] += jp[a] - jm[a];
  }
  const double mu0 = __ldg(ms + c), mu1 = __ldg(ms + F + c);
  double out[N];
  double xi[N];
  xi_of(P, P.step, x + g.x0, y + g.y0, z + g.z0, xi);
  phi_cell<TA>(P, plane_T(P, P, (double)z), ph, gd, divh, mu0, mu1, xi, out);
#pragma unroll
  for (int a = 0; a < N; ++a) pd[a * F + c] = out[a];
}

// ---------------------------------------------------------------------------
// Naive mu-sweep: one thread per cell, 6 faces each (Algorithm 1 line 3).
// ---------------------------------------------------------------------------
template <int L>
__device__ __forceinline__ void load_side(const double* __restrict__ ps, const double* __restrict__ pd,
                                          const double* __restrict__ ms, int64_t F, int64_t c, int64_t s1, int64_t s2,
                                          FaceSide& o) {
#pragma unroll
  for (int a = 0; a < N; ++a) {
    const double* f = ps + a * F;
    o.f[a] = __ldg(f + c);
    o.c1[a] = __ldg(f + c + s1) - __ldg(f + c - s1);
    o.c2[a] = __ldg(f + c + s2) - __ldg(f + c - s2);
  }
#pragma unroll
  for (int s = 0; s < NSOL; ++s) {
    const int a = solid_phase(L, s);
    o.ds[s] = __ldg(pd + a * F + c) - o.f[a];
  }
  o.m[0] = __ldg(ms + c);
  o.m[1] = __ldg(ms + F + c);
}

template <int L, bool TA>
__global__ void __launch_bounds__(256) k_mu_naive(DevParams P, Geom g, const double* __restrict__ ps,
                                                  const double* __restrict__ pd, const double* __restrict__ ms,
                                                  double* __restrict__ md) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const int64_t c = g.at(x, y, z);
  const int64_t F = g.field;
  const double Tc = plane_T(P, P, (double)z);
  double divh[M] = {0.0, 0.0};
#pragma unroll 1
  for (int d = 0; d < 3; ++d) {
    const int64_t sn = d == 0 ? 1 : (d == 1 ? g.pitch : g.plane);
    const int64_t s1 = d == 0 ? g.pitch : 1;
    const int64_t s2 = d == 2 ? g.pitch : g.plane;
    const double Tp = d == 2 ? plane_T(P, P, z + 0.5) : Tc;
    const double Tm = d == 2 ? plane_T(P, P, z - 0.5) : Tc;
    FaceSide sm, s0, sp;
    load_side<L>(ps, pd, ms, F, c - sn, s1, s2, sm);
    load_side<L>(ps, pd, ms, F, c, s1, s2, s0);
    load_side<L>(ps, pd, ms, F, c + sn, s1, s2, sp);
    double Fp[M], Fm[M];
    mu_face<L, TA>(P, Tp, s0, sp, Fp);
    mu_face<L, TA>(P, Tm, sm, s0, Fm);
#pragma unroll
    for (int i = 0; i < M; ++i) divh[i] += Fp[i] - Fm[i];
  }
  double ph[N], dph[N], mu[M], out[M];
#pragma unroll
  for (int a = 0; a < N; ++a) {
    ph[a] = __ldg(ps + a * F + c);
    dph[a] = __ldg(pd + a * F + c) - ph[a];
  }
#pragma unroll
  for (int i = 0; i < M; ++i) mu[i] = __ldg(ms + i * F + c);
  mu_cell<TA>(P, Tc, ph, dph, mu, divh, out);
#pragma unroll
  for (int i = 0; i < M; ++i) md[i * F + c] = out[i];
}

void launch_phi_naive(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                      cudaStream_t s) {
  dim3 b(32, 4, 2), gr((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  PF_DISPATCH(P.liquid, P.TA, (k_phi_naive<LL, TT><<<gr, b, 0, s>>>(P, g, ps, ms, pd)));
}

void launch_mu_naive(const DevParams& P, const Geom& g, const double* ps, const double* pd, const double* ms,
                     double* md, cudaStream_t s) {
  dim3 b(32, 4, 2), gr((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  PF_DISPATCH(P.liquid, P.TA, (k_mu_naive<LL, TT><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md)));
}

// ---------------------------------------------------------------------------
// Split kernels (the paper's "split" variant; Table 1 "partial"):
// a staggered kernel evaluates each face flux once and stores it in a global
// array J[d][comp] (the flux of the face c - e_d / 2, for cells c in
// [0, n] per axis), a cell kernel reads the six fluxes of its cell back.  The
// face and cell arithmetic is the naive kernels', in the same order, so the
// results are bitwise equal to PF_VARIANT_NAIVE.
// ---------------------------------------------------------------------------
template <int L, bool TA>
__global__ void __launch_bounds__(256) k_phi_stag(DevParams P, Geom g, const double* __restrict__ ps,
                                                  double* __restrict__ J) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x > g.nx || y > g.ny || z > g.nz) return;
  const int64_t c = g.at(x, y, z), F = g.field;
  double q[N];
#pragma unroll
  for (int a = 0; a < N; ++a) q[a] = __ldg(ps + a * F + c);
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    const int64_t st = d == 0 ? 1 : (d == 1 ? g.pitch : g.plane);
    double p[N], j[N];
#pragma unroll
    for (int a = 0; a < N; ++a) p[a] = __ldg(ps + a * F + c - st);
    phi_face(P, p, q, j);
#pragma unroll
    for (int a = 0; a < N; ++a) J[(d * N + a) * F + c] = j[a];
  }
}

template <int L, bool TA>
__global__ void __launch_bounds__(256) k_phi_cellsplit(DevParams P, Geom g, const double* __restrict__ ps,
                                                       const double* __restrict__ ms, const double* __restrict__ J,
                                                       double* __restrict__ pd) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const int64_t c = g.at(x, y, z), F = g.field;
  double ph[N], gd[N][3], divh[N] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll
  for (int a = 0; a < N; ++a) ph[a] = __ldg(ps + a * F + c);
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    const int64_t st = d == 0 ? 1 : (d == 1 ? g.pitch : g.plane);
#pragma unroll
    for (int a = 0; a < N; ++a) {
      gd[a][d] = __ldg(ps + a * F + c + st) - __ldg(ps + a * F + c - st);
      divh[a] += __ldg(J + (d * N + a) * F + c + st) - __ldg(J + (d * N + a) * F + c);
    }
  }
  const double mu0 = __ldg(ms + c), mu1 = __ldg(ms + F + c);
  double out[N], xi[N];
  xi_of(P, P.step, x + g.x0, y + g.y0, z + g.z0, xi);
  phi_cell<TA>(P, plane_T(P, P, (double)z), ph, gd, divh, mu0, mu1, xi, out);
#pragma unroll
  for (int a = 0; a < N; ++a) pd[a * F + c] = out[a];
}

template <int L, bool TA>
__global__ void __launch_bounds__(256) k_mu_stag(DevParams P, Geom g, const double* __restrict__ ps,
                                                 const double* __restrict__ pd, const double* __restrict__ ms,
                                                 double* __restrict__ J) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x > g.nx || y > g.ny || z > g.nz) return;
  const int64_t c = g.at(x, y, z), F = g.field;
  const double Tc = plane_T(P, P, (double)z);
#pragma unroll 1
  for (int d = 0; d < 3; ++d) {
    const int64_t sn = d == 0 ? 1 : (d == 1 ? g.pitch : g.plane);
    const int64_t s1 = d == 0 ? g.pitch : 1;
    const int64_t s2 = d == 2 ? g.pitch : g.plane;
    const double Tm = d == 2 ? plane_T(P, P, z - 0.5) : Tc;
    FaceSide sm, s0;
    load_side<L>(ps, pd, ms, F, c - sn, s1, s2, sm);
    load_side<L>(ps, pd, ms, F, c, s1, s2, s0);
    double Fm[M];
    mu_face<L, TA>(P, Tm, sm, s0, Fm);
#pragma unroll
    for (int i = 0; i < M; ++i) J[(d * M + i) * F + c] = Fm[i];
  }
}

template <int L, bool TA>
__global__ void __launch_bounds__(256) k_mu_cellsplit(DevParams P, Geom g, const double* __restrict__ ps,
                                                      const double* __restrict__ pd, const double* __restrict__ ms,
                                                      const double* __restrict__ J, double* __restrict__ md) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z * blockDim.z + threadIdx.z;
  if (x >= g.nx || y >= g.ny || z >= g.nz) return;
  const int64_t c = g.at(x, y, z), F = g.field;
  const double Tc = plane_T(P, P, (double)z);
  double divh[M] = {0.0, 0.0};
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    const int64_t sn = d == 0 ? 1 : (d == 1 ? g.pitch : g.plane);
#pragma unroll
    for (int i = 0; i < M; ++i) divh[i] += __ldg(J + (d * M + i) * F + c + sn) - __ldg(J + (d * M + i) * F + c);
  }
  double ph[N], dph[N], mu[M], out[M];
#pragma unroll
  for (int a = 0; a < N; ++a) {
    ph[a] = __ldg(ps + a * F + c);
    dph[a] = __ldg(pd + a * F + c) - ph[a];
  }
#pragma unroll
  for (int i = 0; i < M; ++i) mu[i] = __ldg(ms + i * F + c);
  mu_cell<TA>(P, Tc, ph, dph, mu, divh, out);
#pragma unroll
  for (int i = 0; i < M; ++i) md[i * F + c] = out[i];
}

void launch_phi_split(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* J, double* pd,
                      cudaStream_t s) {
  dim3 b(32, 4, 2), gs((g.nx + 1 + 31) / 32, (g.ny + 1 + 3) / 4, (g.nz + 1 + 1) / 2),
      gc((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  PF_DISPATCH(P.liquid, P.TA, (k_phi_stag<LL, TT><<<gs, b, 0, s>>>(P, g, ps, J)));
  PF_DISPATCH(P.liquid, P.TA, (k_phi_cellsplit<LL, TT><<<gc, b, 0, s>>>(P, g, ps, ms, J, pd)));
}

void launch_mu_split(const DevParams& P, const Geom& g, const double* ps, const double* pd, const double* ms,
                     double* J, double* md, cudaStream_t s) {
  dim3 b(32, 4, 2), gs((g.nx + 1 + 31) / 32, (g.ny + 1 + 3) / 4, (g.nz + 1 + 1) / 2),
      gc((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  PF_DISPATCH(P.liquid, P.TA, (k_mu_stag<LL, TT><<<gs, b, 0, s>>>(P, g, ps, pd, ms, J)));
  PF_DISPATCH(P.liquid, P.TA, (k_mu_cellsplit<LL, TT><<<gc, b, 0, s>>>(P, g, ps, pd, ms, J, md)));
}

// ---------------------------------------------------------------------------
// Ghost layers (Alg. 1 lines 2 and 4, "communication and boundary handling").
// Every ghost cell is written from interior values by a per-axis index map,
// which equals the ordered x -> y -> z fill (edges and corners consistent,
// SURVEY C.6.6): periodic wrap, Neumann = adjacent interior; a ghost on a
// Dirichlet side gets mu_inf [A15].  Sides with kind -1 are left alone
// (filled by the halo exchange).
// ---------------------------------------------------------------------------
struct GhostArgs {
  Geom g;
  BCSpec bc;
  int ncomp;
  double dir[M];
  int use_dir;
  int vec_x;  // x ghost sectors 32-B aligned (nx % 4 == 0, xoff % 4 == 0): full-sector stores
};

__device__ __forceinline__ int map_axis(int i, int n, int klo, int khi, bool* skip, bool* dirich) {
  if (i < 0) {
    if (klo < 0) { *skip = true; return i; }
    if (klo == PF_BC_DIRICHLET_MU) *dirich = true;
    return klo == PF_BC_PERIODIC ? n - 1 : 0;
  }
  if (i >= n) {
    if (khi < 0) { *skip = true; return i; }
    if (khi == PF_BC_DIRICHLET_MU) *dirich = true;
    return khi == PF_BC_PERIODIC ? 0 : n - 1;
  }
  return i;
}

// One launch fills all ghosts of a field set: blockIdx.y selects the z ghost
// planes (0), the y ghost rows of interior planes (1) or the x ghost columns
// of interior rows (2); 32-bit index math, x fastest (coalesced for 0, 1).
__global__ void k_ghost(GhostArgs A, double* __restrict__ f) {
  const Geom& g = A.g;
  const int sx = g.nx + 2, sy = g.ny + 2;
  const int seg = blockIdx.y;
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  int x, y, z;
  if (seg == 0) {  // 2 planes of sx * sy
    if (i >= 2 * sx * sy) return;
    const int side = i / (sx * sy), r = i - side * sx * sy;
    z = side ? g.nz : -1;
    y = r / sx - 1;
    x = r % sx - 1;
  } else if (seg == 1) {  // 2 rows of sx per interior plane
    if (i >= 2 * sx * g.nz) return;
    const int zz = i / (2 * sx), r = i - zz * 2 * sx;
    z = zz;
    y = (r / sx) ? g.ny : -1;
    x = r % sx - 1;
  } else {  // 2 cells per interior row
    if (i >= 2 * g.ny * g.nz) return;
    const int row = i >> 1;
    z = row / g.ny;
    y = row - z * g.ny;
    x = (i & 1) ? g.nx : -1;
  }
  bool skip = false, dir = false;
  const int mx = map_axis(x, g.nx, A.bc.kind_lo[0], A.bc.kind_hi[0], &skip, &dir);
  const int my = map_axis(y, g.ny, A.bc.kind_lo[1], A.bc.kind_hi[1], &skip, &dir);
  const int mz = map_axis(z, g.nz, A.bc.kind_lo[2], A.bc.kind_hi[2], &skip, &dir);
  if (skip) return;
  const int64_t dst = g.at(x, y, z);
  const int64_t src = g.at(mx, my, mz);
  // all loads first (the source and destination share the array, so a
  // load-store loop would serialise on the possible alias)
  double v[N];
#pragma unroll
  for (int c = 0; c < N; ++c)
    if (c < A.ncomp) v[c] = (dir && A.use_dir) ? A.dir[c < M ? c : 0] : __ldg(f + c * g.field + src);
  if (seg == 2 && A.vec_x) {
    // x ghost columns: store the whole 32-B sector (x = -4..-1, or nx..nx+3)
    // with the ghost value so that L2 never merges a partial sector with
    // DRAM; the other three slots are guard cells that no result depends on
    const int64_t base = g.at(x < 0 ? -4 : g.nx, y, z);
#pragma unroll
    for (int c = 0; c < N; ++c)
      if (c < A.ncomp) {
        double2* q = reinterpret_cast<double2*>(f + c * g.field + base);
        q[0] = make_double2(v[c], v[c]);
        q[1] = make_double2(v[c], v[c]);
      }
    return;
  }
#pragma unroll
  for (int c = 0; c < N; ++c)
    if (c < A.ncomp) f[c * g.field + dst] = v[c];
}

void launch_ghost_fill(const Geom& g, const BCSpec& bc, double* f, int ncomp, const double* dirichlet, cudaStream_t s,
                       bool skip_x) {
  GhostArgs A;
  A.g = g;
  A.bc = bc;
  A.ncomp = ncomp;
  A.use_dir = dirichlet != nullptr;
  for (int i = 0; i < M; ++i) A.dir[i] = dirichlet ? dirichlet[i] : 0.0;
  A.vec_x = (g.nx % 4 == 0 && g.xoff % 4 == 0 && g.pitch % 4 == 0 && g.xoff >= 4 &&
             g.pitch - g.xoff >= (int64_t)g.nx + 4);
  const int64_t n0 = 2 * (int64_t)(g.nx + 2) * (g.ny + 2), n1 = 2 * (int64_t)(g.nx + 2) * g.nz,
                n2 = 2 * (int64_t)g.ny * g.nz;
  const int64_t mx = n0 > n1 ? (n0 > n2 ? n0 : n2) : (n1 > n2 ? n1 : n2);
  // segment 2 (the x ghost columns) is not needed when the sweeps wrap x
  dim3 grid((unsigned)((mx + 255) / 256), skip_x ? 2 : 3);
  k_ghost<<<grid, 256, 0, s>>>(A, f);
}

// ---------------------------------------------------------------------------
// Moving window [A16]: dst(z) = src(z + k) for z + k < nz, else inflow
// (phi = e_l, mu = mu_inf).  Out-of-place; the caller swaps.
// ---------------------------------------------------------------------------
__global__ void k_shift(Geom g, int k, int L, int nph, int nmu, double mi0, double mi1, const double* __restrict__ ps,
                        const double* __restrict__ ms, double* __restrict__ pd, double* __restrict__ md) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y;
  const int z = blockIdx.z;
  if (x >= g.nx) return;
  const int64_t c = g.at(x, y, z);
  const bool in = z + k < g.nz;
  const int64_t sidx = in ? g.at(x, y, z + k) : 0;
  for (int a = 0; a < nph; ++a) pd[a * g.field + c] = in ? ps[a * g.field + sidx] : (a == L ? 1.0 : 0.0);
  md[c] = in ? ms[sidx] : mi0;
  if (nmu > 1) md[g.field + c] = in ? ms[g.field + sidx] : mi1;
}

__global__ void k_set_steps(StepVals* dst, StepBatch b) {
  const int i = threadIdx.x;
  if (i < b.k) {
    dst[i].Tbase = b.Tbase[i];
    dst[i].step = b.step0 + (unsigned long long)i;
  }
}

void launch_set_steps(StepVals* dst, const StepBatch& b, cudaStream_t s) { k_set_steps<<<1, 64, 0, s>>>(dst, b); }

void launch_shift(const Geom& g, int k, int liquid, int nph, int nmu, const double* mu_inf, const double* ps,
                  const double* ms, double* pd, double* md, cudaStream_t s) {
  dim3 b(128), gr((g.nx + 127) / 128, g.ny, g.nz);
  k_shift<<<gr, b, 0, s>>>(g, k, liquid, nph, nmu, mu_inf[0], nmu > 1 ? mu_inf[1] : 0.0, ps, ms, pd, md);
}

// front height: max z with phi_l < 1/2 (deterministic integer max).  One
// block per (y-slab, z) plane: block-level OR, one atomic per block.
__global__ void k_front(Geom g, const double* __restrict__ phl, int* out) {
  const int z = blockIdx.y;
  bool hit = false;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < g.nx * g.ny; i += gridDim.x * blockDim.x) {
    const int y = i / g.nx, x = i - y * g.nx;
    hit |= phl[g.at(x, y, z)] < 0.5;
  }
  if (__syncthreads_or(hit) && threadIdx.x == 0) atomicMax(out, z + g.z0 + 1);  // H + 1
}

void launch_front_height(const Geom& g, int liquid, const double* phi, int* out, cudaStream_t s) {
  int bx = (g.nx * g.ny + 255) / 256;
  if (bx > 64) bx = 64;
  dim3 gr(bx, g.nz);
  k_front<<<gr, 256, 0, s>>>(g, phi + (int64_t)liquid * g.field, out);
}

// monitors: out[0] = max |sum phi - 1|, out[1] = max(-min phi), as
// order-preserving bit patterns; block-level reduction, one atomic per block
__device__ __forceinline__ unsigned long long ord_bits(double v) {
  unsigned long long b = (unsigned long long)__double_as_longlong(v);
  return (b & 0x8000000000000000ull) ? ~b : (b | 0x8000000000000000ull);
}

__global__ void k_monitor(Geom g, int nph, int nmu, const double* __restrict__ ph, const double* __restrict__ mu,
                          unsigned long long* out) {
  const int z = blockIdx.y;
  double e = -1.0, neg = -INFINITY;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < g.nx * g.ny; i += gridDim.x * blockDim.x) {
    const int y = i / g.nx, x = i - y * g.nx;
    const int64_t c = g.at(x, y, z);
    double sum = 0.0, mn = INFINITY, fin = 0.0;  // fin: 0 for finite values, NaN otherwise
    for (int a = 0; a < nph; ++a) {
      const double v = ph[a * g.field + c];
      sum += v;
      mn = fmin(mn, v);
      fin += v - v;
    }
    for (int i2 = 0; i2 < nmu; ++i2) {
      const double v = mu[i2 * g.field + c];
      fin += v - v;
    }
    const double err = fabs(sum - 1.0);
    e = fmax(e, (fin == 0.0 && err <= 1e300) ? err : INFINITY);  // non-finite -> +inf (fmax drops NaN)
    neg = fmax(neg, -mn);
  }
  for (int o = 16; o > 0; o >>= 1) {
    e = fmax(e, __shfl_xor_sync(0xffffffffu, e, o));
    neg = fmax(neg, __shfl_xor_sync(0xffffffffu, neg, o));
  }
  __shared__ double se[8], sn[8];
  if ((threadIdx.x & 31) == 0) {
    se[threadIdx.x >> 5] = e;
    sn[threadIdx.x >> 5] = neg;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < (int)(blockDim.x >> 5); ++w) {
      e = fmax(e, se[w]);
      neg = fmax(neg, sn[w]);
    }
    atomicMax(out, ord_bits(e));
    atomicMax(out + 1, ord_bits(neg));
  }
}

void launch_monitor(const Geom& g, int nph, int nmu, const double* phi, const double* mu, unsigned long long* out2,
                    cudaStream_t s) {
  int bx = (g.nx * g.ny + 255) / 256;
  if (bx > 64) bx = 64;
  dim3 gr(bx, g.nz);
  k_monitor<<<gr, 256, 0, s>>>(g, nph, nmu, phi, mu, out2);
}

// interior <-> packed [comp][z][y][x] copies
__global__ void k_copy(Geom g, int ncomp, const double* __restrict__ src, double* __restrict__ dst, int to_packed) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y, z = blockIdx.z;
  if (x >= g.nx) return;
  const int64_t c = g.at(x, y, z);
  const int64_t pk = ((int64_t)z * g.ny + y) * g.nx + x;
  const int64_t pstride = (int64_t)g.nx * g.ny * g.nz;
  for (int a = 0; a < ncomp; ++a) {
    if (to_packed)
      dst[a * pstride + pk] = src[a * g.field + c];
    else
      dst[a * g.field + c] = src[a * pstride + pk];
  }
}

void launch_copy_interior(const Geom& g, int ncomp, const double* src, double* dst, int to_packed, cudaStream_t s) {
  dim3 b(128), gr((g.nx + 127) / 128, g.ny, g.nz);
  k_copy<<<gr, b, 0, s>>>(g, ncomp, src, dst, to_packed);
}

// ---------------------------------------------------------------------------
// Halo pack / unpack along dimension d for the ordered x -> y -> z exchange:
// the slab covers the interior range of the dimensions after d and the full
// ghosted range of the dimensions before d, so that edge ghosts travel.
// ---------------------------------------------------------------------------
__host__ __device__ inline void slab_dims(const Geom& g, int d, int* n0, int* n1, int* o0, int* o1) {
  // (u, w) = the two other axes in ascending order
  const int n[3] = {g.nx, g.ny, g.nz};
  const int u = d == 0 ? 1 : 0, w = d == 2 ? 1 : 2;
  *n0 = u < d ? n[u] + 2 : n[u];
  *o0 = u < d ? -1 : 0;
  *n1 = w < d ? n[w] + 2 : n[w];
  *o1 = w < d ? -1 : 0;
}

size_t halo_slab_elems(const Geom& g, int d) {
  int n0, n1, o0, o1;
  slab_dims(g, d, &n0, &n1, &o0, &o1);
  return (size_t)n0 * n1;
}

__global__ void k_pack(Geom g, int d, int idx, int ncomp, double* __restrict__ f, double* __restrict__ buf, int unpack) {
  int n0, n1, o0, o1;
  slab_dims(g, d, &n0, &n1, &o0, &o1);
  const int64_t tot = (int64_t)n0 * n1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot; i += (int64_t)gridDim.x * blockDim.x) {
    const int i0 = (int)(i % n0) + o0, i1 = (int)(i / n0) + o1;
    int c[3];
    c[d] = idx;
    c[d == 0 ? 1 : 0] = i0;
    c[d == 2 ? 1 : 2] = i1;
    const int64_t li = g.at(c[0], c[1], c[2]);
    double v[N];
#pragma unroll
    for (int a = 0; a < N; ++a)
      if (a < ncomp) v[a] = unpack ? buf[a * tot + i] : f[a * g.field + li];
#pragma unroll
    for (int a = 0; a < N; ++a)
      if (a < ncomp) {
        if (unpack)
          f[a * g.field + li] = v[a];
        else
          buf[a * tot + i] = v[a];
      }
  }
}

void launch_pack(const Geom& g, int d, int idx, int ncomp, const double* f, double* buf, cudaStream_t s) {
  const size_t tot = halo_slab_elems(g, d);
  int blocks = (int)((tot + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_pack<<<blocks, 256, 0, s>>>(g, d, idx, ncomp, const_cast<double*>(f), buf, 0);
}

// one stage of the ordered ghost fill: the d-ghost slabs (extended ranges of
// the dimensions before d), kinds per side (-1 = leave alone)
__global__ void k_ghost_stage(Geom g, int d, int klo, int khi, int ncomp, double* __restrict__ f, double dir0,
                              double dir1, int use_dir) {
  int n0, n1, o0, o1;
  slab_dims(g, d, &n0, &n1, &o0, &o1);
  const int n[3] = {g.nx, g.ny, g.nz};
  const int64_t tot = (int64_t)n0 * n1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < 2 * tot; i += (int64_t)gridDim.x * blockDim.x) {
    const int side = i >= tot;
    const int kind = side ? khi : klo;
    if (kind < 0) continue;
    const int64_t j = i - side * tot;
    int c[3], s[3];
    c[d == 0 ? 1 : 0] = s[d == 0 ? 1 : 0] = (int)(j % n0) + o0;
    c[d == 2 ? 1 : 2] = s[d == 2 ? 1 : 2] = (int)(j / n0) + o1;
    c[d] = side ? n[d] : -1;
    s[d] = kind == PF_BC_PERIODIC ? (side ? 0 : n[d] - 1) : (side ? n[d] - 1 : 0);
    const bool dirich = kind == PF_BC_DIRICHLET_MU && use_dir;
    const int64_t li = g.at(c[0], c[1], c[2]);
    const int64_t si = g.at(s[0], s[1], s[2]);
    double v[N];
#pragma unroll
    for (int a = 0; a < N; ++a)
      if (a < ncomp) v[a] = dirich ? (a == 0 ? dir0 : dir1) : __ldg(f + a * g.field + si);
#pragma unroll
    for (int a = 0; a < N; ++a)
      if (a < ncomp) f[a * g.field + li] = v[a];
  }
}

void launch_ghost_stage(const Geom& g, int d, int klo, int khi, double* f, int ncomp, const double* dirichlet,
                        cudaStream_t s) {
  const size_t tot = 2 * halo_slab_elems(g, d);
  int blocks = (int)((tot + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_ghost_stage<<<blocks, 256, 0, s>>>(g, d, klo, khi, ncomp, f, dirichlet ? dirichlet[0] : 0.0,
                                       dirichlet ? dirichlet[1] : 0.0, dirichlet != nullptr);
}

void launch_unpack(const Geom& g, int d, int idx, int ncomp, double* f, const double* buf, cudaStream_t s) {
  const size_t tot = halo_slab_elems(g, d);
  int blocks = (int)((tot + 255) / 256);
  if (blocks > 148 * 4) blocks = 148 * 4;
  k_pack<<<blocks, 256, 0, s>>>(g, d, idx, ncomp, f, const_cast<double*>(buf), 1);
}

}  // namespace pf
