// pf_sweeps.cuh -- bodies of the tuned phi- and mu-sweeps for sm_100a,
// templated on the parameter type PT and geometry type GT: run-time structs
// in the generic (nvcc) build, compile-time constants in the specialised
// (NVRTC) build (pf_jit.cu), so both builds run the same source.
//
// Both kernels are bound by the fp64 pipe (Table 1: ~1.5 kFLOP per cell vs
// 96 B of compulsory traffic), so the design goal is to issue
// as few fp64 instructions per cell as possible and to keep the L1/shared
// memory pipe below the fp64 pipe:
//   * a CTA owns a 32 x 8 column tile and marches along z (2.5-D blocking);
//   * every staggered face flux is computed ONCE: each thread computes the
//     -x, -y and +z faces of its cell, the +x / +y faces come from the
//     neighbour thread (warp shuffle / shared memory), and the two faces on
//     the far tile edges are computed by one extra warp each;
//   * the z-face flux is carried in registers to the next plane.
// The paper's "split" kernels cache fluxes in a global staggered array
// (P:L709-721); here they never leave the SM.
#pragma once
#include "pf_model.cuh"

namespace pf {

// software prefetch distance (planes) into L2 / L1 of the z-marching sweeps:
// PF_PREFETCH 0 = off, 1 = L2, 2 = L1
#ifndef PF_PREFETCH
#define PF_PREFETCH 1
#endif
#ifndef PF_MU_ZCARRY  // own cell's phi_src z column carried in registers (8 loads fewer per cell)
#define PF_MU_ZCARRY 1
#endif
#ifndef PF_HALO_L1
#define PF_HALO_L1 1  // halo-ring cells: next plane's new lines prefetched into L1
#endif
#ifndef PF_PHI_UNROLL  // phi-sweep z loop unrolled: the plane rotation (pm <- p0 <- pp) becomes renaming
#define PF_PHI_UNROLL 3
#endif
constexpr int kPhiUnroll = PF_PHI_UNROLL;
#ifndef PF_MU_FXREG  // cell's own -x / -y face fluxes kept in registers for its divergence
#define PF_MU_FXREG 0
#endif
#ifndef PF_MU_QREG  // own cell's D(k) kept in registers from the build (no shared-memory re-read)
#define PF_MU_QREG 0
#endif
#ifndef PF_MU_RPF  // own cell's L1-missing loads issued one plane ahead into registers
#define PF_MU_RPF 1
#endif
#ifndef PF_PREFETCH_D
#define PF_PREFETCH_D 2  // planes ahead
#endif
#ifndef PF_MU_HPIPE  // halo-ring cell's loads for plane k+1 issued at the end of plane k's face phase
#define PF_MU_HPIPE 0
#endif
#ifndef PF_HALO_D  // planes ahead of the halo-ring L1 prefetch (two-rows-per-thread sweep)
#define PF_HALO_D 1
#endif
#ifndef PF_MU_ROT  // mu-sweep: tile rows (and their roles) rotated over the CTA's warps per tile
#define PF_MU_ROT 0
#endif
#ifndef PF_MU_LDHINT  // L1 policy of the mu-sweep's phi_dst / mu loads: 0 default, 1 evict_first, 2 no_allocate,
#define PF_MU_LDHINT 0  // 3 no_allocate + the two-rows sweep's own phi_src(k+2) lines evict_last
#endif
// load of a phi_dst / mu value in the mu-sweep (used by at most the cells of
// one plane: a hint keeps these lines from evicting the reused phi_src lines)
__device__ __forceinline__ double ldh(const double* p) {
#if PF_MU_LDHINT == 1
  double v;
  asm("ld.global.nc.L1::evict_first.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
#elif PF_MU_LDHINT >= 2
  double v;
  asm("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}
// load of an own phi_src line that the x / y differences re-read two planes later
__device__ __forceinline__ double ldkeep(const double* p) {
#if PF_MU_LDHINT == 3
  double v;
  asm("ld.global.nc.L1::evict_last.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}
__device__ __forceinline__ void prefetch_line(const void* p) {
#if PF_PREFETCH == 1
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
#elif PF_PREFETCH == 2
  asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
#else
  (void)p;
#endif
}

constexpr int TX = 32;
constexpr int TY = 8;
#ifndef PF_ZC_PHI
#define PF_ZC_PHI 12
#endif
#ifndef PF_ZC_MU
#define PF_ZC_MU 12
#endif
constexpr int ZC_PHI = PF_ZC_PHI;  // z-chunk per CTA
constexpr int ZC_MU = PF_ZC_MU;
#ifndef PF_MU_TY
#define PF_MU_TY 4  // tile height of the mu-sweep (4: 4 CTAs of 128 threads per SM)
#endif
constexpr int MU_TY = PF_MU_TY;

// ===========================================================================
// phi-sweep (Algorithm 1 line 1): D3C7 of phi_src, D3C1 of mu_src.
// ===========================================================================
#ifndef PF_PHI_FACES6  // every thread computes all six faces of its cell (no flux exchange, no barrier)
#define PF_PHI_FACES6 0
#endif
#ifndef PF_PHI_ZREC
#define PF_PHI_ZREC 0
#endif
#ifndef PF_PHI_PERS  // six-face phi-sweep as a persistent launch (balanced tile-plane shares)
#define PF_PHI_PERS 0
#endif
#ifndef PF_MU_TMEM  // two-rows mu-sweep: the carried side of plane k-1 in tensor memory (TMEM), not registers
#define PF_MU_TMEM 0
#endif
#ifndef PF_MU_HCAR  // two-rows mu-sweep: the halo ring's phi_src z column carried in shared memory
#define PF_MU_HCAR 0
#endif
#ifndef PF_MU_HASYNC  // two-rows mu-sweep: halo ring staged one plane ahead by cp.async (global -> shared)
#define PF_MU_HASYNC 0
#endif
#ifndef PF_MU_XSHFL  // two-rows mu-sweep: own cd_x from the lane neighbours' carried phi_src (shuffles)
#define PF_MU_XSHFL 0
#endif
#ifndef PF_MU_PERS  // two-rows mu-sweep: full launches persistent (balanced tile-plane shares)
#define PF_MU_PERS 0
#endif
#ifndef PF_PHI_XSH  // six-face sweep, +x face taken from the next lane (31 cells per 32-lane row)
#define PF_PHI_XSH 0
#endif
// cells per tile row of the phi-sweep: with PF_PHI_XSH the last lane of a row
// only evaluates the -x face that is the +x face of the lane before it
constexpr int PHI_TXC = PF_PHI_XSH ? TX - 1 : TX;
template <class PT, class GT, int L, bool TA, int PTY = TY, class RT = DevParams>
__device__ __forceinline__ void phi_tuned_body(const PT& P, const RT& R, const GT& g,
                                               const double* __restrict__ ps, const double* __restrict__ ms,
                                               double* __restrict__ pd, int zlo = 0, int zhi = 1 << 30) {
  // [zlo, zhi): planes of this launch (the z-slab schedule, tuning sched = 1;
  // the six-face one-row sweep only); the grid's z-chunks start at zlo
#if PF_PHI_FACES6
  // one tile (bx, by) over planes [z0, z1)
  auto tile = [&](const int bx, const int by, const int z0, const int z1) {
    // The +x / +y face of a cell is the -x / -y face of its neighbour: both
    // threads evaluate phi_face on the same (left, right) operands, so the
    // two values are bitwise equal and the fluxes still telescope.  Costs
    // two extra face evaluations per cell (the neighbour values are loaded
    // for the central differences anyway) and saves the flux exchange, the
    // per-plane barrier and the tile-edge faces.
#if PF_PHI_XSH
    // lane i holds cell x0 + i; lanes 0..30 update their cells, lane 31 (and
    // lanes past the row's end, clamped to the ghost x = nx) only supply the
    // -x face that is the +x face of the lane before them (same operands:
    // bitwise equal to evaluating it there)
    const int xr = bx * PHI_TXC + threadIdx.x, y = by * PTY + threadIdx.y;
    if (y >= g.ny || bx * PHI_TXC >= g.nx) return;  // whole warps: the shuffles need all lanes
    const bool act = xr < g.nx && threadIdx.x < PHI_TXC;
    const int x = min(xr, g.nx);
#else
    const int x = bx * TX + threadIdx.x, y = by * PTY + threadIdx.y;
    if (x >= g.nx || y >= g.ny) return;
    constexpr bool act = true;
#endif
    const i64 F = g.field, SY = g.pitch, SZ = g.plane;
    i64 c = g.at(x, y, z0);
    double pm[N], p0[N], Fzm[N];
#pragma unroll
    for (int a = 0; a < N; ++a) {
      pm[a] = __ldg(ps + a * F + c - SZ);
      p0[a] = __ldg(ps + a * F + c);
    }
    phi_face(P, pm, p0, Fzm);
#pragma unroll kPhiUnroll
    for (int z = z0; z < z1; ++z, c += SZ) {
      if (PF_PREFETCH && z + PF_PREFETCH_D <= z1 + 1) {
#pragma unroll
        for (int a = 0; a < N; ++a) prefetch_line(ps + a * F + c + PF_PREFETCH_D * SZ);
        prefetch_line(ms + c + PF_PREFETCH_D * SZ);
        prefetch_line(ms + F + c + PF_PREFETCH_D * SZ);
      }
      double pp[N], Fzp[N], gd[N][3], divh[N];
      {
        double xm[N], xp[N], ym[N], yp[N], Fa[N], Fb[N];
#pragma unroll
        for (int a = 0; a < N; ++a) {
          const double* f = ps + a * F + c;
          pp[a] = __ldg(f + SZ);
          xm[a] = __ldg(f - 1);
          xp[a] = __ldg(f + 1);
          ym[a] = __ldg(f - SY);
          yp[a] = __ldg(f + SY);
          gd[a][0] = xp[a] - xm[a];
          gd[a][1] = yp[a] - ym[a];
          gd[a][2] = pp[a] - pm[a];
        }
        phi_face(P, xm, p0, Fa);
#if PF_PHI_XSH
#pragma unroll
        for (int a = 0; a < N; ++a) Fb[a] = __shfl_down_sync(0xffffffffu, Fa[a], 1);
#else
        phi_face(P, p0, xp, Fb);
#endif
#pragma unroll
        for (int a = 0; a < N; ++a) divh[a] = Fb[a] - Fa[a];
        phi_face(P, ym, p0, Fa);
        phi_face(P, p0, yp, Fb);
#pragma unroll
        for (int a = 0; a < N; ++a) divh[a] += Fb[a] - Fa[a];
      }
      phi_face(P, p0, pp, Fzp);
#if PF_PHI_ZREC  // -z face recomputed instead of carried (8 registers fewer)
      phi_face(P, pm, p0, Fzm);
#endif
#pragma unroll
      for (int a = 0; a < N; ++a) divh[a] += Fzp[a] - Fzm[a];
      const double mu0 = __ldg(ms + c), mu1 = __ldg(ms + F + c);
      double out[N], xi[N];
      if constexpr (ParamShape<PT>::xi) xi_of(P, R.step, x + g.x0, y + g.y0, z + g.z0, xi);
      phi_cell<TA>(P, plane_T(P, R, (double)z), p0, gd, divh, mu0, mu1, xi, out);
      if (act) {
#pragma unroll
        for (int a = 0; a < N; ++a) pd[a * F + c] = out[a];
#pragma unroll
        for (int a = 0; a < N; ++a) store_x_ghost(g, pd, x, y, z, a, out[a]);
      }
#pragma unroll
      for (int a = 0; a < N; ++a) {
        pm[a] = p0[a];
        p0[a] = pp[a];
        Fzm[a] = Fzp[a];
      }
    }
  };  // tile
#if PF_PHI_PERS
  // persistent launch (tuning phi_pers): gridDim.x CTAs, each a balanced
  // contiguous share of the tile-planes in tile-major order (no partial last
  // wave; a tile column restarts its z-march ~once instead of once per chunk).
  // Warps advance independently (no barrier in this sweep): the share's
  // position is kept per warp in shared memory, not in registers.
  {
    __shared__ long long seg[PTY][2];
    const int ntx = (g.nx + PHI_TXC - 1) / PHI_TXC, nty = (g.ny + PTY - 1) / PTY;
    volatile long long* vs = seg[threadIdx.y];
    if (threadIdx.x == 0) {
      const i64 total = (i64)ntx * nty * g.nz;
      vs[0] = total * blockIdx.x / gridDim.x;
      vs[1] = total * (blockIdx.x + 1) / gridDim.x;
    }
    __syncwarp();
    for (;;) {
      const i64 lo = vs[0], hi = vs[1];
      if (lo >= hi) break;
      const i64 tl = lo / g.nz;
      const int z0 = (int)(lo - tl * g.nz);
      const int z1 = (int)min((i64)g.nz, (i64)z0 + (hi - lo));
      tile((int)(tl % ntx), (int)(tl / ntx), z0, z1);
      __syncwarp();
      if (threadIdx.x == 0) vs[0] = lo + (z1 - z0);
      __syncwarp();
    }
  }
#else
  tile(blockIdx.x, blockIdx.y, zlo + blockIdx.z * ZC_PHI, min(zlo + (int)blockIdx.z * ZC_PHI + ZC_PHI, min(zhi, g.nz)));
#endif
  return;
#endif
  __shared__ double fy[2][N][PTY][TX];  // -y face flux of every thread, by plane parity
  __shared__ double ex[2][N][PTY];      // +x flux on the right tile edge
  __shared__ double ey[2][N][TX];      // +y flux on the top tile edge
  const int lane = threadIdx.x, w = threadIdx.y;
  const int x0 = blockIdx.x * TX, y0 = blockIdx.y * PTY;
  const int x = x0 + lane, y = y0 + w;
  const bool active = x < g.nx && y < g.ny;
  // ragged tiles: clamp to the ghost cell, whose -x / -y face is the +x / +y
  // face of the last interior cell
  const int xc = min(x, g.nx), yc = min(y, g.ny);
  const int z0 = blockIdx.z * ZC_PHI, z1 = min(z0 + ZC_PHI, g.nz);
  const i64 F = g.field, SY = g.pitch, SZ = g.plane;
  // extra faces: warp 0 lanes < PTY: +x face of row `lane`; warp 1: +y face of column `lane`
  i64 ep = 0, eq = 0;  // the two cells of the extra face, at plane z0
  if (w == 0 && lane < PTY) {
    const int ry = min(y0 + lane, g.ny);
    ep = g.at(min(x0 + TX - 1, g.nx), ry, z0);
    eq = g.at(min(x0 + TX, g.nx), ry, z0);
  } else if (w == 1) {
    const int cx = min(x0 + lane, g.nx);
    ep = g.at(cx, min(y0 + PTY - 1, g.ny), z0);
    eq = g.at(cx, min(y0 + PTY, g.ny), z0);
  }
  const bool extra = (w == 0 && lane < PTY) || w == 1;

  i64 c = g.at(xc, yc, z0);
  double pm[N], p0[N], Fzm[N];
#pragma unroll
  for (int a = 0; a < N; ++a) {
    pm[a] = __ldg(ps + a * F + c - SZ);
    p0[a] = __ldg(ps + a * F + c);
  }
  phi_face(P, pm, p0, Fzm);

#pragma unroll kPhiUnroll
  for (int z = z0; z < z1; ++z, c += SZ, ep += SZ, eq += SZ) {
    const int buf = z & 1;
    if (PF_PREFETCH && z + PF_PREFETCH_D <= z1 + 1) {  // own column ahead (<= nz + 1: guard ring)
#pragma unroll
      for (int a = 0; a < N; ++a) prefetch_line(ps + a * F + c + PF_PREFETCH_D * SZ);
      prefetch_line(ms + c + PF_PREFETCH_D * SZ);
      prefetch_line(ms + F + c + PF_PREFETCH_D * SZ);
    }
    double pp[N], Fxm[N], Fym[N], Fzp[N], gd[N][3];
    {
      double xm[N], xp[N], ym[N], yp[N];
#pragma unroll
      for (int a = 0; a < N; ++a) {
        const double* f = ps + a * F + c;
        pp[a] = __ldg(f + SZ);
        xm[a] = __ldg(f - 1);
        xp[a] = __ldg(f + 1);
        ym[a] = __ldg(f - SY);
        yp[a] = __ldg(f + SY);
        gd[a][0] = xp[a] - xm[a];
        gd[a][1] = yp[a] - ym[a];
        gd[a][2] = pp[a] - pm[a];
      }
      phi_face(P, xm, p0, Fxm);
      phi_face(P, ym, p0, Fym);
    }
    phi_face(P, p0, pp, Fzp);
    if (extra) {
      double fa[N], fb[N], fe[N];
#pragma unroll
      for (int a = 0; a < N; ++a) {
        fa[a] = __ldg(ps + a * F + ep);
        fb[a] = __ldg(ps + a * F + eq);
      }
      phi_face(P, fa, fb, fe);
      if (w == 0) {
#pragma unroll
        for (int a = 0; a < N; ++a) ex[buf][a][lane] = fe[a];
      } else {
#pragma unroll
        for (int a = 0; a < N; ++a) ey[buf][a][lane] = fe[a];
      }
    }
#pragma unroll
    for (int a = 0; a < N; ++a) fy[buf][a][w][lane] = Fym[a];
    const double mu0 = __ldg(ms + c), mu1 = __ldg(ms + F + c);
    __syncthreads();
    double divh[N];
#pragma unroll
    for (int a = 0; a < N; ++a) {
      double fxp = __shfl_down_sync(0xffffffffu, Fxm[a], 1);
      if (lane == TX - 1) fxp = ex[buf][a][w];
      const double fyp = (w < PTY - 1) ? fy[buf][a][w + 1][lane] : ey[buf][a][lane];
      divh[a] = ((fxp - Fxm[a]) + (fyp - Fym[a])) + (Fzp[a] - Fzm[a]);
    }
    double out[N], xi[N];
    if constexpr (ParamShape<PT>::xi) xi_of(P, R.step, x + g.x0, y + g.y0, z + g.z0, xi);
    phi_cell<TA>(P, plane_T(P, R, (double)z), p0, gd, divh, mu0, mu1, xi, out);
    if (active) {
#pragma unroll
      for (int a = 0; a < N; ++a) pd[a * F + c] = out[a];
#pragma unroll
      for (int a = 0; a < N; ++a) store_x_ghost(g, pd, x, y, z, a, out[a]);
    }
#pragma unroll
    for (int a = 0; a < N; ++a) {
      pm[a] = p0[a];
      p0[a] = pp[a];
      Fzm[a] = Fzp[a];
    }
  }
}

// ===========================================================================
// phi-sweep with two tile rows per thread (pf_tuning phi_rpt = 2; six-face
// scheme): thread (lane, w) updates rows y = y0 + 2w and y + 1.  The face
// between the two rows is evaluated once (it is the +y face of the lower and
// the -y face of the upper row, on the same operands as in the one-row
// sweep, so the bits are the same), and each row's y-neighbour inside the
// pair is the other row's phi_src, in registers (no load).
// ===========================================================================
template <class PT, class GT, int L, bool TA, int PTY, class RT = DevParams>
__device__ __forceinline__ void phi_r2_body(const PT& P, const RT& R, const GT& g,
                                            const double* __restrict__ ps, const double* __restrict__ ms,
                                            double* __restrict__ pd, int = 0, int = 0) {  // (full launches only)
  static_assert(PTY % 2 == 0, "phi_rpt = 2 needs an even tile height");
  const int x = blockIdx.x * TX + threadIdx.x, y = blockIdx.y * PTY + 2 * threadIdx.y;
  if (x >= g.nx || y >= g.ny) return;
  const bool act1 = y + 1 < g.ny;  // upper row inside the block (else: the ghost row, not stored)
  const int z0 = blockIdx.z * ZC_PHI, z1 = min(z0 + ZC_PHI, g.nz);
  const i64 F = g.field, SY = g.pitch, SZ = g.plane;
  // upper row's +y neighbour row; clamped to the ghost row when the upper row
  // is itself the ghost row (its update is not stored)
  const i64 SYU = act1 ? SY : 0;
  i64 c = g.at(x, y, z0);
  double pm[2][N], p0[2][N], Fzm[2][N];
#pragma unroll
  for (int a = 0; a < N; ++a) {
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      pm[r][a] = __ldg(ps + a * F + c + r * SY - SZ);
      p0[r][a] = __ldg(ps + a * F + c + r * SY);
    }
  }
  phi_face(P, pm[0], p0[0], Fzm[0]);
  phi_face(P, pm[1], p0[1], Fzm[1]);
#pragma unroll kPhiUnroll
  for (int z = z0; z < z1; ++z, c += SZ) {
    if (PF_PREFETCH && z + PF_PREFETCH_D <= z1 + 1) {
#pragma unroll
      for (int r = 0; r < 2; ++r) {
#pragma unroll
        for (int a = 0; a < N; ++a) prefetch_line(ps + a * F + c + r * SY + PF_PREFETCH_D * SZ);
        prefetch_line(ms + c + r * SY + PF_PREFETCH_D * SZ);
        prefetch_line(ms + F + c + r * SY + PF_PREFETCH_D * SZ);
      }
    }
    double pp[2][N], divh[2][N], gd[2][N][3];
    {
      double xm[N], xp[N], yo[N], Fa[N], Fb[N], Fym[N], Fmid[N];
      // lower row: -x, +x, -y (sums in the one-row sweep's order:
      // divh = ((F+x - F-x) + (F+y - F-y)) + (F+z - F-z))
#pragma unroll
      for (int a = 0; a < N; ++a) {
        const double* f = ps + a * F + c;
        pp[0][a] = __ldg(f + SZ);
        xm[a] = __ldg(f - 1);
        xp[a] = __ldg(f + 1);
        yo[a] = __ldg(f - SY);
        gd[0][a][0] = xp[a] - xm[a];
        gd[0][a][1] = p0[1][a] - yo[a];
        gd[0][a][2] = pp[0][a] - pm[0][a];
      }
      phi_face(P, xm, p0[0], Fa);
      phi_face(P, p0[0], xp, Fb);
#pragma unroll
      for (int a = 0; a < N; ++a) divh[0][a] = Fb[a] - Fa[a];
      phi_face(P, yo, p0[0], Fym);
      // the face between the rows: +y of the lower, -y of the upper row
      phi_face(P, p0[0], p0[1], Fmid);
#pragma unroll
      for (int a = 0; a < N; ++a) divh[0][a] += Fmid[a] - Fym[a];
      // upper row: -x, +x, +y
#pragma unroll
      for (int a = 0; a < N; ++a) {
        const double* f = ps + a * F + c + SY;
        pp[1][a] = __ldg(f + SZ);
        xm[a] = __ldg(f - 1);
        xp[a] = __ldg(f + 1);
        yo[a] = __ldg(f + SYU);
        gd[1][a][0] = xp[a] - xm[a];
        gd[1][a][1] = yo[a] - p0[0][a];
        gd[1][a][2] = pp[1][a] - pm[1][a];
      }
      phi_face(P, xm, p0[1], Fa);
      phi_face(P, p0[1], xp, Fb);
#pragma unroll
      for (int a = 0; a < N; ++a) divh[1][a] = Fb[a] - Fa[a];
      phi_face(P, p0[1], yo, Fb);
#pragma unroll
      for (int a = 0; a < N; ++a) divh[1][a] += Fb[a] - Fmid[a];
    }
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      double Fzp[N];
      phi_face(P, p0[r], pp[r], Fzp);
#pragma unroll
      for (int a = 0; a < N; ++a) divh[r][a] += Fzp[a] - Fzm[r][a];
      const i64 cr = c + r * SY;
      const double mu0 = __ldg(ms + cr), mu1 = __ldg(ms + F + cr);
      double out[N], xi[N];
      if constexpr (ParamShape<PT>::xi) xi_of(P, R.step, x + g.x0, y + r + g.y0, z + g.z0, xi);
      phi_cell<TA>(P, plane_T(P, R, (double)z), p0[r], gd[r], divh[r], mu0, mu1, xi, out);
      if (r == 0 || act1) {
#pragma unroll
        for (int a = 0; a < N; ++a) pd[a * F + cr] = out[a];
#pragma unroll
        for (int a = 0; a < N; ++a) store_x_ghost(g, pd, x, y + r, z, a, out[a]);
      }
#pragma unroll
      for (int a = 0; a < N; ++a) {
        pm[r][a] = p0[r][a];
        p0[r][a] = pp[r][a];
        Fzm[r][a] = Fzp[a];
      }
    }
  }
}

// ===========================================================================
// mu-sweep (Algorithm 1 line 3): D3C19 of phi_src, D3C7 of phi_dst and mu.
//
// Per plane k every cell of the tile and of its 1-cell halo ring publishes
// its "face side" data D (phi, the three central differences, dphi, mu) to
// shared memory once; the -x / -y faces read both sides from there, the
// z-face k-1/2 pairs the previous plane's D (registers) with the current
// one, and the cell update of plane k-1 is done as soon as that z-face is
// known (one-plane lag).
// ===========================================================================
// halo tile of an MTX x MTY column tile (MTX, MTY: tile width and height of the mu-sweep)
template <int MTY, int MTX = TX>
struct MuTile {
  static constexpr int HX = MTX + 2, HY = MTY + 2, NC = HX * HY;
};
// shared-memory D layout, structure of arrays over the NC halo-tile cells
constexpr int D_F = 0;            // phi      [N]
constexpr int D_CX = D_F + N;     // cd_x     [N]
constexpr int D_CY = D_CX + N;    // cd_y     [N]
constexpr int D_CZ = D_CY + N;    // cd_z     [N]
constexpr int D_DP = D_CZ + N;    // dphi     [N] (phi_dst - phi_src)
constexpr int D_MU = D_DP + N;    // mu       [M]
constexpr int D_NV = D_MU + M;    // 22 doubles per cell
template <int MTY, int MTX = TX>
__host__ __device__ constexpr size_t mu_smem_bytes() {
  return (size_t)(D_NV * MuTile<MTY, MTX>::NC + M * MTY * (MTX + 1) + M * (MTY + 1) * MTX) * sizeof(double);
}
// halo-tile coords (0..HX-1, 0..HY-1) -> slot
template <int MTX = TX>
__device__ __forceinline__ int hidx(int hx, int hy) { return hy * (MTX + 2) + hx; }

// D is stored cell-major (array of structures, D_NV = 22 doubles = 176 B per
// cell): the 16-B vector accesses of a warp then fall on distinct bank groups
// (176 = 11 x 16, odd), and a face side is read with 9 LDS.128.

// build D of cell (x,y,k) from global memory into shared slot i;
// wx / wy / wz: compute cd_x / cd_y / cd_z (halo cells only need the
// tangential ones, and must not read beyond the guard ring)
template <int NC, class GT>
__device__ __forceinline__ void build_cell(const GT& g, const double* __restrict__ ps, const double* __restrict__ pd,
                                           const double* __restrict__ ms, int x, int y, int k, bool wx, bool wy,
                                           bool wz, double* __restrict__ D, int i) {
  const i64 F = g.field;
  const i64 c = g.at(x, y, k);
  double v[D_NV];
#pragma unroll
  for (int a = 0; a < N; ++a) {
    const double* f = ps + a * F + c;
    v[D_F + a] = __ldg(f);
    v[D_CX + a] = wx ? __ldg(f + 1) - __ldg(f - 1) : 0.0;
    v[D_CY + a] = wy ? __ldg(f + g.pitch) - __ldg(f - g.pitch) : 0.0;
    v[D_CZ + a] = wz ? __ldg(f + g.plane) - __ldg(f - g.plane) : 0.0;
    v[D_DP + a] = ldh(pd + a * F + c) - v[D_F + a];
  }
  v[D_MU + 0] = ldh(ms + c);
  v[D_MU + 1] = ldh(ms + F + c);
  double2* d = reinterpret_cast<double2*>(D + (size_t)i * D_NV);
#pragma unroll
  for (int j = 0; j < D_NV / 2; ++j) d[j] = make_double2(v[2 * j], v[2 * j + 1]);
}

// halo-ring cell of the mu-sweep, software-pipelined (PF_MU_HPIPE): the raw
// values of plane k+1 are loaded at the end of plane k's face phase (the
// loads complete under the barrier and the next own-cell build) and turned
// into D at plane k+1.  Same arithmetic as build_cell (bitwise equal).
struct HaloRaw {
  double f[N], tp[N], tm[N], zp[N], zm[N], d[N], m[M];
};
template <class GT>
__device__ __forceinline__ void halo_load(const GT& g, const double* __restrict__ ps, const double* __restrict__ pd,
                                          const double* __restrict__ ms, int x, int y, int k, i64 toff, HaloRaw& h) {
  const i64 F = g.field;
  const i64 c = g.at(x, y, k);
#pragma unroll
  for (int a = 0; a < N; ++a) {
    const double* f = ps + a * F + c;
    h.f[a] = __ldg(f);
    h.tp[a] = __ldg(f + toff);
    h.tm[a] = __ldg(f - toff);
    h.zp[a] = __ldg(f + g.plane);
    h.zm[a] = __ldg(f - g.plane);
    h.d[a] = ldh(pd + a * F + c);
  }
  h.m[0] = ldh(ms + c);
  h.m[1] = ldh(ms + F + c);
}
__device__ __forceinline__ void halo_store(const HaloRaw& h, bool wx, double* __restrict__ D, int i) {
  double v[D_NV];
#pragma unroll
  for (int a = 0; a < N; ++a) {
    const double t = h.tp[a] - h.tm[a];
    v[D_F + a] = h.f[a];
    v[D_CX + a] = wx ? t : 0.0;
    v[D_CY + a] = wx ? 0.0 : t;
    v[D_CZ + a] = h.zp[a] - h.zm[a];
    v[D_DP + a] = h.d[a] - h.f[a];
  }
  v[D_MU + 0] = h.m[0];
  v[D_MU + 1] = h.m[1];
  double2* d = reinterpret_cast<double2*>(D + (size_t)i * D_NV);
#pragma unroll
  for (int j = 0; j < D_NV / 2; ++j) d[j] = make_double2(v[2 * j], v[2 * j + 1]);
}

// build D of the own cell (x,y,k) into slot i with its z column carried in
// registers: fc = phi_src(k) (loaded as the +z neighbour one plane earlier),
// fm = phi_src(k-1); loads phi_src(k+1) into fc for the next plane.
template <int NC, class GT>
__device__ __forceinline__ void build_own_carry(const GT& g, const double* __restrict__ ps,
                                                const double* __restrict__ pd, const double* __restrict__ ms, int x,
                                                int y, int k, bool wz, const double (&fm)[N], double (&fc)[N],
                                                double* __restrict__ D, int i, double (&v)[D_NV]) {
  const i64 F = g.field;
  const i64 c = g.at(x, y, k);
#pragma unroll
  for (int a = 0; a < N; ++a) {
    const double* f = ps + a * F + c;
    const double fp = wz ? __ldg(f + g.plane) : 0.0;
    v[D_F + a] = fc[a];
    v[D_CX + a] = __ldg(f + 1) - __ldg(f - 1);
    v[D_CY + a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
    v[D_CZ + a] = wz ? fp - fm[a] : 0.0;
    v[D_DP + a] = ldh(pd + a * F + c) - fc[a];
    fc[a] = fp;
  }
  v[D_MU + 0] = ldh(ms + c);
  v[D_MU + 1] = ldh(ms + F + c);
  double2* d = reinterpret_cast<double2*>(D + (size_t)i * D_NV);
#pragma unroll
  for (int j = 0; j < D_NV / 2; ++j) d[j] = make_double2(v[2 * j], v[2 * j + 1]);
}

// as build_own_carry, with the loads that miss L1 (phi_src(k+1), phi_dst(k),
// mu(k)) taken from registers loaded one plane earlier (nf, nd, nm); the
// loads for plane k+1 are issued here, a whole face phase before their use
template <int NC, class GT>
__device__ __forceinline__ void build_own_rpf(const GT& g, const double* __restrict__ ps,
                                              const double* __restrict__ pd, const double* __restrict__ ms, int x,
                                              int y, int k, bool wz, const double (&fm)[N], double (&fc)[N],
                                              double (&nf)[N], double (&nd)[N], double (&nm)[M],
                                              double* __restrict__ D, int i, double (&v)[D_NV]) {
  const i64 F = g.field;
  const i64 c = g.at(x, y, k);
#pragma unroll
  for (int a = 0; a < N; ++a) {
    const double* f = ps + a * F + c;
    v[D_F + a] = fc[a];
    v[D_CX + a] = __ldg(f + 1) - __ldg(f - 1);
    v[D_CY + a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
    v[D_CZ + a] = wz ? nf[a] - fm[a] : 0.0;
    v[D_DP + a] = nd[a] - fc[a];
    fc[a] = nf[a];
  }
  v[D_MU + 0] = nm[0];
  v[D_MU + 1] = nm[1];
  double2* d = reinterpret_cast<double2*>(D + (size_t)i * D_NV);
#pragma unroll
  for (int j = 0; j < D_NV / 2; ++j) d[j] = make_double2(v[2 * j], v[2 * j + 1]);
  // next plane: only while the march continues (wz == false on the peeled
  // last plane k = z1, where k + 2 could pass the guard ring)
  if (wz) {
#pragma unroll
    for (int a = 0; a < N; ++a) {
      nf[a] = __ldg(ps + a * F + c + 2 * g.plane);
      nd[a] = ldh(pd + a * F + c + g.plane);
    }
    nm[0] = ldh(ms + c + g.plane);
    nm[1] = ldh(ms + F + c + g.plane);
  }
}

template <bool B>
struct BoolC {
  static constexpr bool value = B;
};

template <int L, int NC>
__device__ __forceinline__ void side_from_smem(const double* __restrict__ D, int i, int c1, int c2, FaceSide& s) {
  // (c1, c2: offsets of the two tangential central differences in D)
  const double2* d = reinterpret_cast<const double2*>(D + (size_t)i * D_NV);
  double2 t;
#pragma unroll
  for (int j = 0; j < N / 2; ++j) {
    t = d[(D_F >> 1) + j];
    s.f[2 * j] = t.x;
    s.f[2 * j + 1] = t.y;
    t = d[(c1 >> 1) + j];
    s.c1[2 * j] = t.x;
    s.c1[2 * j + 1] = t.y;
    t = d[(c2 >> 1) + j];
    s.c2[2 * j] = t.x;
    s.c2[2 * j + 1] = t.y;
  }
  double dp[N];
#pragma unroll
  for (int j = 0; j < N / 2; ++j) {
    t = d[(D_DP >> 1) + j];
    dp[2 * j] = t.x;
    dp[2 * j + 1] = t.y;
  }
#pragma unroll
  for (int u = 0; u < NSOL; ++u) s.ds[u] = dp[solid_phase(L, u)];
  t = d[D_MU >> 1];
  s.m[0] = t.x;
  s.m[1] = t.y;
}

// ---------------------------------------------------------------------------
// Thread-block clusters stacked along y (PF tuning knob mu_cly = CLY > 1):
// the CLY tiles of a cluster march z in lockstep (one cluster barrier per
// barrier of the plane) and read each other's shared memory (DSMEM), so an
// interior tile edge builds no y-halo row (its sides are the neighbour's own
// tile row) and its +y edge face flux is the neighbour's -y face flux.
// ---------------------------------------------------------------------------
__device__ __forceinline__ unsigned cl_rank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// shared::cluster address of the same shared-memory object in CTA `rank`
__device__ __forceinline__ unsigned cl_map(const void* p, unsigned rank) {
  const unsigned a = (unsigned)__cvta_generic_to_shared(p);
  unsigned r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
  return r;
}
__device__ __forceinline__ double2 ld_cl2(unsigned a) {
  double2 v;
  asm volatile("ld.shared::cluster.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ double ld_cl(unsigned a) {
  double v;
  asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(a));
  return v;
}
// all threads of all CTAs of the cluster; release/acquire orders the shared
// memory writes before it with the (remote) reads after it
__device__ __forceinline__ void cl_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// side_from_smem of a slot in another CTA's D (a = its shared::cluster address)
template <int L>
__device__ __forceinline__ void side_from_cl(unsigned a, int c1, int c2, FaceSide& s) {
  double2 t;
#pragma unroll
  for (int j = 0; j < N / 2; ++j) {
    t = ld_cl2(a + 8u * (D_F + 2 * j));
    s.f[2 * j] = t.x;
    s.f[2 * j + 1] = t.y;
    t = ld_cl2(a + 8u * (c1 + 2 * j));
    s.c1[2 * j] = t.x;
    s.c1[2 * j + 1] = t.y;
    t = ld_cl2(a + 8u * (c2 + 2 * j));
    s.c2[2 * j] = t.x;
    s.c2[2 * j + 1] = t.y;
  }
  double dp[N];
#pragma unroll
  for (int j = 0; j < N / 2; ++j) {
    t = ld_cl2(a + 8u * (D_DP + 2 * j));
    dp[2 * j] = t.x;
    dp[2 * j + 1] = t.y;
  }
#pragma unroll
  for (int u = 0; u < NSOL; ++u) s.ds[u] = dp[solid_phase(L, u)];
  t = ld_cl2(a + 8u * D_MU);
  s.m[0] = t.x;
  s.m[1] = t.y;
}

template <class PT, class GT, int L, bool TA, int MTY, int MTX = TX, int CLY = 1, class RT = DevParams>
__device__ __forceinline__ void mu_tuned_body(const PT& P, const RT& R, const GT& g, const TileSel& ts,
                                              const double* __restrict__ ps, const double* __restrict__ pd,
                                              const double* __restrict__ ms, double* __restrict__ md) {
  constexpr int NC = MuTile<MTY, MTX>::NC, HX = MuTile<MTY, MTX>::HX;
  static_assert(2 * MTX + 2 * MTY <= MTY * MTX, "the halo ring needs 2 MTX + 2 MTY threads");
  static_assert(MTX % 16 == 0 && MTX <= 32, "tile rows of whole 128-B lines");
  const int tbx = blockIdx.x + ts.off[0], tby = blockIdx.y + ts.off[1], tbz = blockIdx.z + ts.off[2];
  if (ts.skip && tbx >= ts.lo[0] && tbx < ts.hi[0] && tby >= ts.lo[1] && tby < ts.hi[1] && tbz >= ts.lo[2] &&
      tbz < ts.hi[2])
    return;  // interior tile, done by the other launch
  extern __shared__ double smem[];
  double* D = smem;                          // [NC][D_NV] (AoS: LDS.128 per pair)
  double* fxs = D + D_NV * NC;               // [M][MTY][MTX+1]: x-face fluxes, face i = x0 - 1/2 + i
  double* fys = fxs + M * MTY * (MTX + 1);    // [M][MTY+1][MTX]: y-face fluxes
  // lane: x in the tile, w: row.  With PF_MU_ROT the row of hardware warp
  // threadIdx.y is rotated by a hash of the tile: warp i of every CTA sits on
  // SM sub-partition i, and the extra jobs of a plane (halo rows, far-edge
  // faces) belong to fixed rows, so without rotation the same sub-partitions
  // would carry them in every CTA
  int w = threadIdx.y;
  if (PF_MU_ROT && MTX == 32) {
    const unsigned bid = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    w = (int)((threadIdx.y + ((bid * 0x9E3779B1u) >> 16)) % (unsigned)MTY);
  }
  const int lane = threadIdx.x, t = w * MTX + lane;
  const int x0 = tbx * MTX, y0 = tby * MTY;
  const int x = x0 + lane, y = y0 + w;
  const bool active = x < g.nx && y < g.ny;
  const int xc = min(x, g.nx), yc = min(y, g.ny);
  const int z0 = tbz * ZC_MU, z1 = min(z0 + ZC_MU, g.nz);
  const i64 F = g.field;
  const int me = hidx<MTX>(lane + 1, w + 1);
  // halo ring cell owned by thread t >= MTX MTY - (2 MTX + 2 MTY) (corners
  // are not needed): the last threads build the halo ring, the first ones
  // compute the far-edge faces.  The x-halo cells come first so that with
  // 32-wide tiles each halo row is built by one whole warp (a warp's loads
  // then touch the lines of one row, not of two rows and a column).
  int hx = 0, hy = 0, hs = -1;
  bool hwx = false, hwy = false;
  const int th = t - (MTY * MTX - (2 * MTX + 2 * MTY));
  if (th >= 0 && th < MTY) { hx = 0; hy = th + 1; hwy = true; }
  else if (th >= MTY && th < 2 * MTY) { hx = MTX + 1; hy = th - MTY + 1; hwy = true; }
  else if (th >= 2 * MTY && th < 2 * MTY + MTX) { hx = th - 2 * MTY + 1; hy = 0; hwx = true; }
  else if (th >= 2 * MTY + MTX && th < 2 * MTY + 2 * MTX) { hx = th - 2 * MTY - MTX + 1; hy = MTY + 1; hwx = true; }
  if (hwx || hwy) hs = hidx<MTX>(hx, hy);
  // cluster mode: the y-halo row of an edge shared with a tile of the same
  // cluster is that tile's own row (read through DSMEM), not built here
  constexpr bool CL = CLY > 1;
  static_assert(!CL || MTX == 32, "cluster mode needs 32-wide tiles");
  // (the cluster rank and the DSMEM addresses are re-read where used: fewer
  // live registers across the march)
  if constexpr (CL) {
    const unsigned cr = cl_rank();
    if ((hy == 0 && hwx && cr > 0) || (hy == MTY + 1 && hwx && cr + 1 < (unsigned)CLY)) hs = -1;
  }
  const int hgx = min(x0 + hx - 1, g.nx), hgy = min(y0 + hy - 1, g.ny);
  // far-edge face of thread t: t < MTX: +y face of the top tile row, column t;
  // MTX <= t < MTX + MTY: +x face of the right tile column, row t - MTX.
  // One code path for both (slots and tangential components per thread), so
  // that a warp holding both kinds computes them in one pass.
  const bool eyf = t < MTX, exf = t >= MTX && t < MTX + MTY;
  const int ep = eyf ? hidx<MTX>(t + 1, MTY) : hidx<MTX>(MTX, t - MTX + 1);
  const int eq = eyf ? hidx<MTX>(t + 1, MTY + 1) : hidx<MTX>(MTX + 1, t - MTX + 1);
  const int ec1 = eyf ? D_CX : D_CY;
  const int eo = eyf ? (MTY * MTX + t) : (t - MTX) * (MTX + 1) + MTX;  // flux slot (component 0)
  double* const eout = eyf ? fys : fxs;
  const int estr = eyf ? (MTY + 1) * MTX : MTY * (MTX + 1);           // component stride

  // z-face k-1/2 needs the previous plane's side (tangential: x, y)
  FaceSide Dp;
  double dpl = 0.0;  // dphi of the liquid at plane k-1 (for the cell update)
  {
    const i64 c = g.at(xc, yc, z0 - 1);
#pragma unroll
    for (int a = 0; a < N; ++a) {
      const double* f = ps + a * F + c;
      Dp.f[a] = __ldg(f);
      Dp.c1[a] = __ldg(f + 1) - __ldg(f - 1);
      Dp.c2[a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
    }
#pragma unroll
    for (int s = 0; s < NSOL; ++s) {
      const int a = solid_phase(L, s);
      Dp.ds[s] = ldh(pd + a * F + c) - Dp.f[a];
    }
    Dp.m[0] = ldh(ms + c);
    Dp.m[1] = ldh(ms + F + c);
  }
  double divxy[M] = {0.0, 0.0}, Fzm[M] = {0.0, 0.0};
#if PF_MU_HPIPE
  HaloRaw hraw;
  const i64 htoff = hwx ? 1 : g.pitch;  // the halo cell's tangential direction
  if (hs >= 0 && z0 < z1) halo_load(g, ps, pd, ms, hgx, hgy, z0, htoff, hraw);
#endif
#if PF_MU_ZCARRY
  double fcar[N];  // phi_src(k) of the own cell, carried along z
  {
    const i64 c = g.at(xc, yc, z0);
#pragma unroll
    for (int a = 0; a < N; ++a) fcar[a] = __ldg(ps + a * F + c);
  }
#endif
#if PF_MU_RPF
  double rnf[N], rnd[N], rnm[M];  // phi_src(k+1), phi_dst(k), mu(k) of the own cell
  {
    const i64 c = g.at(xc, yc, z0);
#pragma unroll
    for (int a = 0; a < N; ++a) {
      rnf[a] = __ldg(ps + a * F + c + g.plane);
      rnd[a] = ldh(pd + a * F + c);
    }
    rnm[0] = ldh(ms + c);
    rnm[1] = ldh(ms + F + c);
  }
#endif

  // one plane of the march; the last one (k = z1) only completes the cell
  // updates of plane z1 - 1, peeled so that the main loop has no such tests
  auto plane = [&](auto lastc, const int k) {
    constexpr bool last = decltype(lastc)::value;
    if (PF_PREFETCH && k + PF_PREFETCH_D <= z1 + 1) {  // own cell's lines of the next planes
      const i64 cp = g.at(xc, yc, k);
#pragma unroll
      for (int a = 0; a < N; ++a) {
        prefetch_line(ps + a * F + cp + PF_PREFETCH_D * g.plane);
        prefetch_line(pd + a * F + cp + (PF_PREFETCH_D - 1) * g.plane);
      }
      prefetch_line(ms + cp + (PF_PREFETCH_D - 1) * g.plane);
      prefetch_line(ms + F + cp + (PF_PREFETCH_D - 1) * g.plane);
    }
    if (PF_HALO_L1 && !last && hs >= 0) {  // halo-ring cell's lines of the next plane into L1
      const i64 ch = g.at(hgx, hgy, k + 1);
#pragma unroll
      for (int a = 0; a < N; ++a) {
        asm volatile("prefetch.global.L1 [%0];" ::"l"(ps + a * F + ch + g.plane));
        asm volatile("prefetch.global.L1 [%0];" ::"l"(pd + a * F + ch));
      }
      asm volatile("prefetch.global.L1 [%0];" ::"l"(ms + ch));
      asm volatile("prefetch.global.L1 [%0];" ::"l"(ms + F + ch));
    }
    // (a) publish D(k) of the own cell and of the halo ring
    double vo[D_NV];  // own cell's D(k) (kept in registers with PF_MU_QREG)
#if PF_MU_RPF
    build_own_rpf<NC>(g, ps, pd, ms, xc, yc, k, !last, Dp.f, fcar, rnf, rnd, rnm, D, me, vo);
#elif PF_MU_ZCARRY
    build_own_carry<NC>(g, ps, pd, ms, xc, yc, k, !last, Dp.f, fcar, D, me, vo);
#else
    build_cell<NC>(g, ps, pd, ms, xc, yc, k, true, true, !last, D, me);
#endif
#if PF_MU_HPIPE
    if (!last && hs >= 0) halo_store(hraw, hwx, D, hs);
#else
    if (!last && hs >= 0) build_cell<NC>(g, ps, pd, ms, hgx, hgy, k, hwx, hwy, true, D, hs);
#endif
    if constexpr (CL)
      cl_sync();
    else
      __syncthreads();
    // (b) z-face k-1/2 from registers (plane k-1) and shared memory (plane k)
    FaceSide q;
#if PF_MU_QREG && (PF_MU_RPF || PF_MU_ZCARRY)
#pragma unroll
    for (int a = 0; a < N; ++a) {
      q.f[a] = vo[D_F + a];
      q.c1[a] = vo[D_CX + a];
      q.c2[a] = vo[D_CY + a];
    }
#pragma unroll
    for (int u = 0; u < NSOL; ++u) q.ds[u] = vo[D_DP + solid_phase(L, u)];
    q.m[0] = vo[D_MU];
    q.m[1] = vo[D_MU + 1];
#else
    side_from_smem<L, NC>(D, me, D_CX, D_CY, q);
#endif
    double Fz[M];
    mu_face<L, TA>(P, plane_T(P, R, k - 0.5), Dp, q, Fz);
    // (c) cell update of plane k-1
    if (k > z0 && active) {
      double ph[N], dph[N], out[M];
      const double divh[M] = {divxy[0] + (Fz[0] - Fzm[0]), divxy[1] + (Fz[1] - Fzm[1])};
#pragma unroll
      for (int a = 0; a < N; ++a) ph[a] = Dp.f[a];
#pragma unroll
      for (int s = 0; s < NSOL; ++s) dph[solid_phase(L, s)] = Dp.ds[s];
      dph[L] = dpl;
      mu_cell<TA>(P, plane_T(P, R, (double)(k - 1)), ph, dph, Dp.m, divh, out);
      const i64 c = g.at(xc, yc, k - 1);
      md[c] = out[0];
      md[F + c] = out[1];
    }
    Fzm[0] = Fz[0];
    Fzm[1] = Fz[1];
    // carry plane k's side for the next z-face
    Dp = q;
#if PF_MU_QREG && (PF_MU_RPF || PF_MU_ZCARRY)
    dpl = vo[D_DP + L];
#else
    dpl = D[(size_t)me * D_NV + D_DP + L];
#endif
    double Fx[M], Fy[M];  // -x / -y face fluxes of the own cell, plane k
    if constexpr (!last) {
      // (d) faces of plane k: -x and -y of every thread, + the far tile edges
      const double Tk = plane_T(P, R, (double)k);
      // (the own side is Dp = plane k's {f, cx, cy, ds, mu}, already in
      // registers: only its cz comes from shared memory)
      FaceSide p, s;
#if PF_MU_QREG && (PF_MU_RPF || PF_MU_ZCARRY)
#pragma unroll
      for (int a = 0; a < N; ++a) s.c2[a] = vo[D_CZ + a];
#else
      {
        const double2* d = reinterpret_cast<const double2*>(D + (size_t)me * D_NV + D_CZ);
        const double2 z01 = d[0], z23 = d[1];
        s.c2[0] = z01.x; s.c2[1] = z01.y; s.c2[2] = z23.x; s.c2[3] = z23.y;
      }
#endif
#pragma unroll
      for (int a = 0; a < N; ++a) {
        s.f[a] = Dp.f[a];
        s.c1[a] = Dp.c2[a];
      }
#pragma unroll
      for (int u = 0; u < NSOL; ++u) s.ds[u] = Dp.ds[u];
      s.m[0] = Dp.m[0];
      s.m[1] = Dp.m[1];
      side_from_smem<L, NC>(D, me - 1, D_CY, D_CZ, p);
      mu_face<L, TA>(P, Tk, p, s, Fx);
#pragma unroll
      for (int a = 0; a < N; ++a) s.c1[a] = Dp.c1[a];
      if (CL && w == 0 && cl_rank() > 0)  // the tile below's top row, column `lane`
        side_from_cl<L>(cl_map(D + (size_t)hidx<MTX>(lane + 1, MTY) * D_NV, cl_rank() - 1), D_CX, D_CZ, p);
      else
        side_from_smem<L, NC>(D, me - HX, D_CX, D_CZ, p);
      mu_face<L, TA>(P, Tk, p, s, Fy);
#pragma unroll
      for (int i = 0; i < M; ++i) {
        fxs[(i * MTY + w) * (MTX + 1) + lane] = Fx[i];
        fys[(i * (MTY + 1) + w) * MTX + lane] = Fy[i];
      }
      if constexpr (MTX == 32) {  // far tile edges in different warps: compile-time components
        if (w == 0 && !(CL && cl_rank() + 1 < (unsigned)CLY)) {  // +y face of the top tile edge, column `lane`
          double Fe[M];
          side_from_smem<L, NC>(D, hidx<MTX>(lane + 1, MTY), D_CX, D_CZ, p);
          side_from_smem<L, NC>(D, hidx<MTX>(lane + 1, MTY + 1), D_CX, D_CZ, s);
          mu_face<L, TA>(P, Tk, p, s, Fe);
#pragma unroll
          for (int i = 0; i < M; ++i) fys[(i * (MTY + 1) + MTY) * MTX + lane] = Fe[i];
        } else if (w == 1 && lane < MTY) {  // +x face of the right tile edge, row `lane`
          double Fe[M];
          side_from_smem<L, NC>(D, hidx<MTX>(MTX, lane + 1), D_CY, D_CZ, p);
          side_from_smem<L, NC>(D, hidx<MTX>(MTX + 1, lane + 1), D_CY, D_CZ, s);
          mu_face<L, TA>(P, Tk, p, s, Fe);
#pragma unroll
          for (int i = 0; i < M; ++i) fxs[(i * MTY + lane) * (MTX + 1) + MTX] = Fe[i];
        }
      } else if (eyf || exf) {  // both kinds in one warp: one pass
        double Fe[M];
        side_from_smem<L, NC>(D, ep, ec1, D_CZ, p);
        side_from_smem<L, NC>(D, eq, ec1, D_CZ, s);
        mu_face<L, TA>(P, Tk, p, s, Fe);
#pragma unroll
        for (int i = 0; i < M; ++i) eout[eo + i * estr] = Fe[i];
      }
    }
    if constexpr (!last) {
#if PF_MU_HPIPE
      if (hs >= 0 && k + 1 < z1) halo_load(g, ps, pd, ms, hgx, hgy, k + 1, htoff, hraw);
#endif
      if constexpr (CL)
        cl_sync();
      else
        __syncthreads();
      // (cluster mode: the top row's +y flux is the -y flux of the tile above)
      double fyu[M];
#pragma unroll
      for (int i = 0; i < M; ++i)
        fyu[i] = (CL && w == MTY - 1 && cl_rank() + 1 < (unsigned)CLY)  // row 0 of the tile above
                     ? ld_cl(cl_map(fys + i * (MTY + 1) * MTX + lane, cl_rank() + 1))
                     : fys[(i * (MTY + 1) + w + 1) * MTX + lane];
#pragma unroll
      for (int i = 0; i < M; ++i)
#if PF_MU_FXREG  // own -x / -y fluxes from registers, only the +x / +y ones from shared memory
        divxy[i] = (fxs[(i * MTY + w) * (MTX + 1) + lane + 1] - Fx[i]) + (fyu[i] - Fy[i]);
#else
        divxy[i] = (fxs[(i * MTY + w) * (MTX + 1) + lane + 1] - fxs[(i * MTY + w) * (MTX + 1) + lane]) +
                   (fyu[i] - fys[(i * (MTY + 1) + w) * MTX + lane]);
#endif
    }
  };
  for (int k = z0; k < z1; ++k) plane(BoolC<false>{}, k);
  plane(BoolC<true>{}, z1);
}


#if PF_MU_TMEM
// ---------------------------------------------------------------------------
// Tensor memory (TMEM, 256 KB per SM, tcgen05.*) as per-thread scratch from
// SIMT code: the 17 doubles of a face side (f, c1, c2, ds, m) as 34 columns
// of the thread's TMEM lane (a warp accesses the 32 lanes of its quarter).
// tools/tmem_probe.cu measured the round trip on a B200.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void tm_st_side(unsigned ta, const FaceSide& s) {
  unsigned u[34];
  double v[17];
#pragma unroll
  for (int a = 0; a < N; ++a) { v[a] = s.f[a]; v[4 + a] = s.c1[a]; v[8 + a] = s.c2[a]; }
#pragma unroll
  for (int t = 0; t < NSOL; ++t) v[12 + t] = s.ds[t];
  v[15] = s.m[0];
  v[16] = s.m[1];
#pragma unroll
  for (int i = 0; i < 17; ++i) { u[2 * i] = (unsigned)__double2loint(v[i]); u[2 * i + 1] = (unsigned)__double2hiint(v[i]); }
  asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31, %32};\n" ::"r"(ta), "r"(u[0]), "r"(u[1]), "r"(u[2]), "r"(u[3]), "r"(u[4]), "r"(u[5]), "r"(u[6]), "r"(u[7]), "r"(u[8]), "r"(u[9]), "r"(u[10]), "r"(u[11]), "r"(u[12]), "r"(u[13]), "r"(u[14]), "r"(u[15]), "r"(u[16]), "r"(u[17]), "r"(u[18]), "r"(u[19]), "r"(u[20]), "r"(u[21]), "r"(u[22]), "r"(u[23]), "r"(u[24]), "r"(u[25]), "r"(u[26]), "r"(u[27]), "r"(u[28]), "r"(u[29]), "r"(u[30]), "r"(u[31]) : "memory");
  asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};\n" ::"r"(ta + 32u), "r"(u[32]), "r"(u[33]) : "memory");
}
__device__ __forceinline__ void tm_ld_side(unsigned ta, FaceSide& s) {
  unsigned u[34];
  asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];\n" : "=r"(u[0]), "=r"(u[1]), "=r"(u[2]), "=r"(u[3]), "=r"(u[4]), "=r"(u[5]), "=r"(u[6]), "=r"(u[7]), "=r"(u[8]), "=r"(u[9]), "=r"(u[10]), "=r"(u[11]), "=r"(u[12]), "=r"(u[13]), "=r"(u[14]), "=r"(u[15]), "=r"(u[16]), "=r"(u[17]), "=r"(u[18]), "=r"(u[19]), "=r"(u[20]), "=r"(u[21]), "=r"(u[22]), "=r"(u[23]), "=r"(u[24]), "=r"(u[25]), "=r"(u[26]), "=r"(u[27]), "=r"(u[28]), "=r"(u[29]), "=r"(u[30]), "=r"(u[31]) : "r"(ta) : "memory");
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x2.b32 {%0, %1}, [%2];\n" : "=r"(u[32]), "=r"(u[33]) : "r"(ta + 32u) : "memory");
  asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
  double v[17];
#pragma unroll
  for (int i = 0; i < 17; ++i) v[i] = __hiloint2double((int)u[2 * i + 1], (int)u[2 * i]);
#pragma unroll
  for (int a = 0; a < N; ++a) { s.f[a] = v[a]; s.c1[a] = v[4 + a]; s.c2[a] = v[8 + a]; }
#pragma unroll
  for (int t = 0; t < NSOL; ++t) s.ds[t] = v[12 + t];
  s.m[0] = v[15];
  s.m[1] = v[16];
}
#endif
// asynchronous global -> shared copies (cp.async, sm_80+): 8 B cached in L1
// (.ca), 16 B cached in L2 only (.cg); completion per thread (wait_all), a
// CTA barrier after it publishes the data to the other threads
__device__ __forceinline__ void cp_async8(void* smem, const void* gmem) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"((unsigned)__cvta_generic_to_shared(smem)),
               "l"(gmem)
               : "memory");
}
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"((unsigned)__cvta_generic_to_shared(smem)),
               "l"(gmem)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// ===========================================================================
// mu-sweep with two tile rows per thread (pf_tuning mu_rpt = 2): a CTA of
// 32 x (MTY/2) threads owns a 32 x MTY tile; thread (lane, w) updates rows
// 2w and 2w+1.  Per cell this halves the y-halo ring (2 halo rows per MTY
// rows), the barriers and the far-edge faces, and the y-face between a
// thread's two rows takes both sides from registers.  Same per-face and
// per-cell arithmetic as mu_tuned_body, so the two give the same bits.
// ===========================================================================
template <class PT, class GT, int L, bool TA, int MTY, class RT = DevParams>
__device__ __forceinline__ void mu_r2_body(const PT& P, const RT& R, const GT& g, const TileSel& ts,
                                           const double* __restrict__ ps, const double* __restrict__ pd,
                                           const double* __restrict__ ms, double* __restrict__ md) {
  constexpr int MTX = 32, TYT = MTY / 2, NT = MTX * TYT;
  constexpr int NC = MuTile<MTY, MTX>::NC, HX = MuTile<MTY, MTX>::HX;
  static_assert(MTY % 2 == 0 && 2 * MTX + 2 * MTY <= NT && TYT >= 2, "mu_rpt = 2 needs an even MTY >= 6");
  // one tile column (tbx, tby) over planes [z0, z1)
  auto tile = [&](const int tbx, const int tby, const int z0, const int z1) {
  extern __shared__ double smem[];
  double* D = smem;
  double* fxs = D + D_NV * NC;             // [M][MTY][MTX+1]
  double* fys = fxs + M * MTY * (MTX + 1);  // [M][MTY+1][MTX]
  const int lane = threadIdx.x, w = threadIdx.y, t = w * MTX + lane;
  const int x0 = tbx * MTX, y0 = tby * MTY;
  const int x = x0 + lane;
  const i64 F = g.field;
  const int xc = min(x, g.nx);
  int yc[2], me[2];
  bool active[2];
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int y = y0 + 2 * w + r;
    active[r] = x < g.nx && y < g.ny;
    yc[r] = min(y, g.ny);
    me[r] = hidx<MTX>(lane + 1, 2 * w + r + 1);
  }
  // halo ring: the last 2 MTX + 2 MTY threads, x-halo cells first
  int hx = 0, hy = 0, hs = -1;
  bool hwx = false, hwy = false;
  const int th = t - (NT - (2 * MTX + 2 * MTY));
  if (th >= 0 && th < MTY) { hx = 0; hy = th + 1; hwy = true; }
  else if (th >= MTY && th < 2 * MTY) { hx = MTX + 1; hy = th - MTY + 1; hwy = true; }
  else if (th >= 2 * MTY && th < 2 * MTY + MTX) { hx = th - 2 * MTY + 1; hy = 0; hwx = true; }
  else if (th >= 2 * MTY + MTX && th < 2 * MTY + 2 * MTX) { hx = th - 2 * MTY - MTX + 1; hy = MTY + 1; hwx = true; }
  if (hwx || hwy) hs = hidx<MTX>(hx, hy);
  const int hgx = min(x0 + hx - 1, g.nx), hgy = min(y0 + hy - 1, g.ny);
#if PF_MU_HCAR || PF_MU_HASYNC
  // halo ring with its phi_src z column carried in shared memory (tuning
  // mu_hcar): ring cell ci holds phi_src of planes k-1, k, k+1 in slots
  // (k+2)%3, k%3, (k+1)%3, so a halo cell loads per plane only phi_src(k+1),
  // the solids' phi_dst and mu (9 loads instead of 26; the 2 x MTY column
  // cells are 16 lines per warp load).  Its tangential and z differences
  // come from the ring: the same operands, so the same bits as build_cell.
  // Ring order: left column (hy = 0..MTY+1), right column, bottom row
  // (hx = 1..MTX), top row; the 4 corners are carried by threads 0..3.
  constexpr int RC = 2 * (MTY + 2) + 2 * MTX;
  static_assert(NT - 2 * MTX - 2 * MTY >= 4, "mu_hcar: four free threads carry the ring corners");
#if PF_MU_HASYNC != 2
  __shared__ __align__(16) double fring[3][N][RC];  // phase-major: a warp's ring reads are contiguous
#endif
  auto ridx = [](int rx, int ry) {
    return rx == 0 ? ry : rx == MTX + 1 ? MTY + 2 + ry : 2 * (MTY + 2) + (ry == 0 ? 0 : MTX) + rx - 1;
  };
  int ci = -1, tpi = 0, tmi = 0;
  i64 cring = 0;
  if (hs >= 0) {
    ci = ridx(hx, hy);
    tpi = hwx ? ridx(hx + 1, hy) : ridx(hx, hy + 1);
    tmi = hwx ? ridx(hx - 1, hy) : ridx(hx, hy - 1);
    cring = g.at(hgx, hgy, 0);
  } else if (t < 4) {
    const int chx = (t & 1) ? MTX + 1 : 0, chy = (t & 2) ? MTY + 1 : 0;
    ci = ridx(chx, chy);
    cring = g.at(min(x0 + chx - 1, g.nx), min(y0 + chy - 1, g.ny), 0);
  }
#if PF_MU_HASYNC
  // tuning mu_hasync: the ring is filled by asynchronous copies (cp.async)
  // one build ahead -- per plane k, after the barrier that ends the build of
  // D(k), phi_src(k + 2) into ring slot (k + 2) % 3 (the slot of k - 1, just
  // read) and the solids' phi_dst / mu of plane k + 1 into dring, completed
  // before the plane's second barrier -- so a halo cell builds its side with
  // no global load on the critical path
  __shared__ __align__(16) double dring[NSOL + M][RC];
#if PF_MU_HASYNC == 2
  // mu_hasync 2: the whole halo tile's phi_src planes (rows x0 - 2 .. x0 +
  // MTX + 1, 16-B pieces cached in L2 only; rows are 128-B aligned) in a
  // 3-plane ring: the own cells take phi_src(k) and its x / y / z neighbours
  // from shared memory as well (only phi_dst and mu of the own cells stay
  // register-prefetched loads).  Past the ghost cell of a ragged tile the
  // pieces hold what memory holds there (only inactive cells read those).
  constexpr int TRX = MTX + 4, TRP = TRX / 2;  // ring row length, 16-B pieces per row
  __shared__ __align__(16) double tring[3][N][MTY + 2][TRX];
#endif
  auto stage = [&](const int kf, const int kd) {
#if PF_MU_HASYNC == 2
    for (int it = t; it < (MTY + 2) * N * TRP; it += NT) {
      const int pc = it % TRP, a = (it / TRP) % N, ry = it / (TRP * N);
      cp_async16(&tring[(kf + 3) % 3][a][ry][2 * pc],
                 ps + a * F + g.at(x0 - 2 + 2 * pc, min(y0 + ry - 1, g.ny), kf));
    }
#else
    if (ci >= 0) {
#pragma unroll
      for (int a = 0; a < N; ++a) cp_async8(&fring[(kf + 3) % 3][a][ci], ps + a * F + cring + (i64)kf * g.plane);
    }
#endif
    if (kd >= 0 && hs >= 0) {
#pragma unroll
      for (int u = 0; u < NSOL; ++u)
        cp_async8(&dring[u][ci], pd + solid_phase(L, u) * F + cring + (i64)kd * g.plane);
#pragma unroll
      for (int i = 0; i < M; ++i) cp_async8(&dring[NSOL + i][ci], ms + i * F + cring + (i64)kd * g.plane);
    }
    cp_async_commit();
  };
  stage(z0 - 1, -1);
  stage(z0, -1);
  stage(z0 + 1, z0);
  cp_async_wait_all();
#else
  if (ci >= 0) {
    const double* f = ps + cring + (i64)(z0 - 1) * g.plane;
#pragma unroll
    for (int a = 0; a < N; ++a) {
      fring[(z0 + 2) % 3][a][ci] = __ldg(f + a * F);
      fring[z0 % 3][a][ci] = __ldg(f + a * F + g.plane);
    }
  }
#endif
  __syncthreads();
#endif

  FaceSide Dp[2];
  double dpl[2] = {0.0, 0.0};
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const i64 c = g.at(xc, yc[r], z0 - 1);
#pragma unroll
    for (int a = 0; a < N; ++a) {
      const double* f = ps + a * F + c;
      Dp[r].f[a] = __ldg(f);
      Dp[r].c1[a] = __ldg(f + 1) - __ldg(f - 1);
      Dp[r].c2[a] = __ldg(f + g.pitch) - __ldg(f - g.pitch);
    }
#pragma unroll
    for (int s = 0; s < NSOL; ++s) {
      const int a = solid_phase(L, s);
      Dp[r].ds[s] = ldh(pd + a * F + c) - Dp[r].f[a];
    }
    Dp[r].m[0] = ldh(ms + c);
    Dp[r].m[1] = ldh(ms + F + c);
  }
#if PF_MU_TMEM
  // the carried side of plane k-1 lives in TMEM between planes (68 columns
  // of this thread's lane: row r at column 34 r); only its phi_src (the z
  // central difference of the build) stays in registers
  __shared__ unsigned tm_base;
  if (w == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;\n" ::"r"(
                     (unsigned)__cvta_generic_to_shared(&tm_base)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n");
  }
  asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
  const unsigned tm = tm_base + ((unsigned)(32 * (w & 3)) << 16);
  double fprev[2][N];
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    tm_st_side(tm + 34u * r, Dp[r]);
#pragma unroll
    for (int a = 0; a < N; ++a) fprev[r][a] = Dp[r].f[a];
  }
#endif
  double divxy[2][M] = {{0.0, 0.0}, {0.0, 0.0}}, Fzm[2][M] = {{0.0, 0.0}, {0.0, 0.0}};
  double fcar[2][N];
#if PF_MU_RPF
  double rnf[2][N], rnd[2][N], rnm[2][M];
#endif
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const i64 c = g.at(xc, yc[r], z0);
#pragma unroll
    for (int a = 0; a < N; ++a) fcar[r][a] = __ldg(ps + a * F + c);
#if PF_MU_RPF
#pragma unroll
    for (int a = 0; a < N; ++a) {
      rnf[r][a] = __ldg(ps + a * F + c + g.plane);
      rnd[r][a] = ldh(pd + a * F + c);
    }
    rnm[r][0] = ldh(ms + c);
    rnm[r][1] = ldh(ms + F + c);
#endif
  }

  auto plane = [&](auto lastc, const int k) {
    constexpr bool last = decltype(lastc)::value;
    if (PF_PREFETCH && k + PF_PREFETCH_D <= z1 + 1) {
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const i64 cp = g.at(xc, yc[r], k);
#pragma unroll
        for (int a = 0; a < N; ++a) {
          prefetch_line(ps + a * F + cp + PF_PREFETCH_D * g.plane);
          prefetch_line(pd + a * F + cp + (PF_PREFETCH_D - 1) * g.plane);
        }
        prefetch_line(ms + cp + (PF_PREFETCH_D - 1) * g.plane);
        prefetch_line(ms + F + cp + (PF_PREFETCH_D - 1) * g.plane);
      }
    }
    if (PF_HALO_L1 && !last && hs >= 0 && k + PF_HALO_D <= z1) {  // halo lines PF_HALO_D planes ahead
      const i64 ch = g.at(hgx, hgy, k + PF_HALO_D);
#pragma unroll
      for (int a = 0; a < N; ++a) {
        asm volatile("prefetch.global.L1 [%0];" ::"l"(ps + a * F + ch + g.plane));
        asm volatile("prefetch.global.L1 [%0];" ::"l"(pd + a * F + ch));
      }
      asm volatile("prefetch.global.L1 [%0];" ::"l"(ms + ch));
      asm volatile("prefetch.global.L1 [%0];" ::"l"(ms + F + ch));
    }
    // (a) publish D(k) of the two own cells and of the halo ring
#if PF_MU_HASYNC == 2 && PF_MU_RPF
    {
      // mu_hasync 2: phi_src(k) and its neighbours from the staged tile ring
      // (the operands of the register path below: the same bits); phi_dst
      // and mu of the own cells register-prefetched one plane ahead
      const int s0 = k % 3, sp = (k + 1) % 3, sm = (k + 2) % 3;
      double v0[D_NV], v1[D_NV];
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        double* v = r ? v1 : v0;
        const int ry = 2 * w + r + 1;
#pragma unroll
        for (int a = 0; a < N; ++a) {
          v[D_F + a] = tring[s0][a][ry][lane + 2];
          v[D_CX + a] = tring[s0][a][ry][lane + 3] - tring[s0][a][ry][lane + 1];
          v[D_CY + a] = tring[s0][a][ry + 1][lane + 2] - tring[s0][a][ry - 1][lane + 2];
          v[D_CZ + a] = !last ? tring[sp][a][ry][lane + 2] - tring[sm][a][ry][lane + 2] : 0.0;
          v[D_DP + a] = rnd[r][a] - v[D_F + a];
        }
        v[D_MU] = rnm[r][0];
        v[D_MU + 1] = rnm[r][1];
      }
      double2* d0 = reinterpret_cast<double2*>(D + (size_t)me[0] * D_NV);
      double2* d1 = reinterpret_cast<double2*>(D + (size_t)me[1] * D_NV);
#pragma unroll
      for (int j = 0; j < D_NV / 2; ++j) {
        d0[j] = make_double2(v0[2 * j], v0[2 * j + 1]);
        d1[j] = make_double2(v1[2 * j], v1[2 * j + 1]);
      }
#pragma unroll
      for (int r = 0; r < 2 && !last; ++r) {
        const i64 c = g.at(xc, yc[r], k);
#pragma unroll
        for (int a = 0; a < N; ++a) rnd[r][a] = ldh(pd + a * F + c + g.plane);
        rnm[r][0] = ldh(ms + c + g.plane);
        rnm[r][1] = ldh(ms + F + c + g.plane);
      }
    }
#elif PF_MU_RPF
    {
      // as build_own_rpf for both rows; each row's y-neighbour inside the
      // pair is the other row's carried phi_src(k) (for an active row it is
      // the value at that address; an inactive row's cd_y is never read)
      const i64 c0 = g.at(xc, yc[0], k), c1 = g.at(xc, yc[1], k);
      double v0[D_NV], v1[D_NV];
#pragma unroll
      for (int a = 0; a < N; ++a) {
        const double* f0 = ps + a * F + c0;
        const double* f1 = ps + a * F + c1;
        v0[D_F + a] = fcar[0][a];
        v1[D_F + a] = fcar[1][a];
#if PF_MU_XSHFL
        {
          // phi_src(k) of the x-neighbours is the neighbour lane's carried
          // value; lanes 0 / 31 load the halo column's (the same operands)
          const bool edge = lane == 0 || lane == MTX - 1;
          const int eo = lane == 0 ? -1 : 1;
          const double e0 = edge ? __ldg(f0 + eo) : 0.0, e1 = edge ? __ldg(f1 + eo) : 0.0;
          const double u0 = __shfl_up_sync(0xffffffffu, fcar[0][a], 1), d0 = __shfl_down_sync(0xffffffffu, fcar[0][a], 1);
          const double u1 = __shfl_up_sync(0xffffffffu, fcar[1][a], 1), d1 = __shfl_down_sync(0xffffffffu, fcar[1][a], 1);
          v0[D_CX + a] = (lane == MTX - 1 ? e0 : d0) - (lane == 0 ? e0 : u0);
          v1[D_CX + a] = (lane == MTX - 1 ? e1 : d1) - (lane == 0 ? e1 : u1);
        }
#else
        v0[D_CX + a] = __ldg(f0 + 1) - __ldg(f0 - 1);
        v1[D_CX + a] = __ldg(f1 + 1) - __ldg(f1 - 1);
#endif
        v0[D_CY + a] = fcar[1][a] - __ldg(f0 - g.pitch);
        v1[D_CY + a] = __ldg(f1 + g.pitch) - fcar[0][a];
#if PF_MU_TMEM
        v0[D_CZ + a] = !last ? rnf[0][a] - fprev[0][a] : 0.0;
        v1[D_CZ + a] = !last ? rnf[1][a] - fprev[1][a] : 0.0;
#else
        v0[D_CZ + a] = !last ? rnf[0][a] - Dp[0].f[a] : 0.0;
        v1[D_CZ + a] = !last ? rnf[1][a] - Dp[1].f[a] : 0.0;
#endif
        v0[D_DP + a] = rnd[0][a] - fcar[0][a];
        v1[D_DP + a] = rnd[1][a] - fcar[1][a];
      }
#pragma unroll
      for (int a = 0; a < N; ++a) {
        fcar[0][a] = rnf[0][a];
        fcar[1][a] = rnf[1][a];
      }
      v0[D_MU] = rnm[0][0];
      v0[D_MU + 1] = rnm[0][1];
      v1[D_MU] = rnm[1][0];
      v1[D_MU + 1] = rnm[1][1];
      double2* d0 = reinterpret_cast<double2*>(D + (size_t)me[0] * D_NV);
      double2* d1 = reinterpret_cast<double2*>(D + (size_t)me[1] * D_NV);
#pragma unroll
      for (int j = 0; j < D_NV / 2; ++j) {
        d0[j] = make_double2(v0[2 * j], v0[2 * j + 1]);
        d1[j] = make_double2(v1[2 * j], v1[2 * j + 1]);
      }
      // next plane (not on the peeled last plane k = z1, where k + 2 could
      // pass the guard ring)
#pragma unroll
      for (int r = 0; r < 2 && !last; ++r) {
        const i64 c = r ? c1 : c0;
#pragma unroll
        for (int a = 0; a < N; ++a) {
          rnf[r][a] = ldkeep(ps + a * F + c + 2 * g.plane);
          rnd[r][a] = ldh(pd + a * F + c + g.plane);
        }
        rnm[r][0] = ldh(ms + c + g.plane);
        rnm[r][1] = ldh(ms + F + c + g.plane);
      }
    }
#else
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      double vo[D_NV];
#if PF_MU_RPF
      build_own_rpf<NC>(g, ps, pd, ms, xc, yc[r], k, !last, Dp[r].f, fcar[r], rnf[r], rnd[r], rnm[r], D, me[r], vo);
#elif PF_MU_TMEM
      build_own_carry<NC>(g, ps, pd, ms, xc, yc[r], k, !last, fprev[r], fcar[r], D, me[r], vo);
#else
      build_own_carry<NC>(g, ps, pd, ms, xc, yc[r], k, !last, Dp[r].f, fcar[r], D, me[r], vo);
#endif
    }
#endif
#if PF_MU_HASYNC
    if (!last && hs >= 0) {  // the side from the staged ring (the operands of build_cell: the same bits)
      const int sm = (k + 2) % 3, s0 = k % 3, sp = (k + 1) % 3;
      double v[D_NV];
#pragma unroll
      for (int a = 0; a < N; ++a) {
#if PF_MU_HASYNC == 2
        const double tt = hwx ? tring[s0][a][hy][hx + 2] - tring[s0][a][hy][hx]
                              : tring[s0][a][hy + 1][hx + 1] - tring[s0][a][hy - 1][hx + 1];
        v[D_F + a] = tring[s0][a][hy][hx + 1];
        v[D_CZ + a] = tring[sp][a][hy][hx + 1] - tring[sm][a][hy][hx + 1];
#else
        const double tt = fring[s0][a][tpi] - fring[s0][a][tmi];
        v[D_F + a] = fring[s0][a][ci];
        v[D_CZ + a] = fring[sp][a][ci] - fring[sm][a][ci];
#endif
        v[D_CX + a] = hwx ? tt : 0.0;
        v[D_CY + a] = hwx ? 0.0 : tt;
        v[D_DP + a] = 0.0;  // the liquid's dphi of a halo cell is never read
      }
#pragma unroll
      for (int u = 0; u < NSOL; ++u) {
        const int a = solid_phase(L, u);
        v[D_DP + a] = dring[u][ci] - v[D_F + a];
      }
      v[D_MU + 0] = dring[NSOL][ci];
      v[D_MU + 1] = dring[NSOL + 1][ci];
      double2* d = reinterpret_cast<double2*>(D + (size_t)hs * D_NV);
#pragma unroll
      for (int j = 0; j < D_NV / 2; ++j) d[j] = make_double2(v[2 * j], v[2 * j + 1]);
    }
#elif PF_MU_HCAR
    if (!last && ci >= 0) {
      const i64 c = cring + (i64)k * g.plane;
      const int sm = (k + 2) % 3, s0 = k % 3, sp = (k + 1) % 3;
      double fn[N];
#pragma unroll
      for (int a = 0; a < N; ++a) fn[a] = __ldg(ps + a * F + c + g.plane);
      if (hs >= 0) {
        double v[D_NV];
#pragma unroll
        for (int a = 0; a < N; ++a) {
          const double tt = fring[s0][a][tpi] - fring[s0][a][tmi];
          v[D_F + a] = fring[s0][a][ci];
          v[D_CX + a] = hwx ? tt : 0.0;
          v[D_CY + a] = hwx ? 0.0 : tt;
          v[D_CZ + a] = fn[a] - fring[sm][a][ci];
          v[D_DP + a] = 0.0;  // the liquid's dphi of a halo cell is never read
        }
#pragma unroll
        for (int u = 0; u < NSOL; ++u) {
          const int a = solid_phase(L, u);
          v[D_DP + a] = ldh(pd + a * F + c) - v[D_F + a];
        }
        v[D_MU + 0] = ldh(ms + c);
        v[D_MU + 1] = ldh(ms + F + c);
        double2* d = reinterpret_cast<double2*>(D + (size_t)hs * D_NV);
#pragma unroll
        for (int j = 0; j < D_NV / 2; ++j) d[j] = make_double2(v[2 * j], v[2 * j + 1]);
      }
#pragma unroll
      for (int a = 0; a < N; ++a) fring[sp][a][ci] = fn[a];
    }
#else
    if (!last && hs >= 0) build_cell<NC>(g, ps, pd, ms, hgx, hgy, k, hwx, hwy, true, D, hs);
#endif
    __syncthreads();
#if PF_MU_HASYNC
    if (!last && k + 1 < z1) stage(k + 2, k + 1);  // the next build's ring (overwrites what this build read)
#endif
    // (b) z-faces k-1/2 and (c) cell updates of plane k-1
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      FaceSide q;
      side_from_smem<L, NC>(D, me[r], D_CX, D_CY, q);
#if PF_MU_TMEM
      tm_ld_side(tm + 34u * r, Dp[r]);
#endif
      double Fz[M];
      mu_face<L, TA>(P, plane_T(P, R, k - 0.5), Dp[r], q, Fz);
      if (k > z0 && active[r]) {
        double ph[N], dph[N], out[M];
        const double divh[M] = {divxy[r][0] + (Fz[0] - Fzm[r][0]), divxy[r][1] + (Fz[1] - Fzm[r][1])};
#pragma unroll
        for (int a = 0; a < N; ++a) ph[a] = Dp[r].f[a];
#pragma unroll
        for (int s = 0; s < NSOL; ++s) dph[solid_phase(L, s)] = Dp[r].ds[s];
        dph[L] = dpl[r];
        mu_cell<TA>(P, plane_T(P, R, (double)(k - 1)), ph, dph, Dp[r].m, divh, out);
        const i64 c = g.at(xc, yc[r], k - 1);
        md[c] = out[0];
        md[F + c] = out[1];
      }
      Fzm[r][0] = Fz[0];
      Fzm[r][1] = Fz[1];
#if PF_MU_TMEM
      if constexpr (!last) {
        tm_st_side(tm + 34u * r, q);
#pragma unroll
        for (int a = 0; a < N; ++a) fprev[r][a] = q.f[a];
      }
#else
      Dp[r] = q;
#endif
      dpl[r] = D[(size_t)me[r] * D_NV + D_DP + L];
    }
    if constexpr (!last) {
      // (d) faces of plane k: -x of both rows, -y of the lower row (from
      // shared memory), the y-face between the two rows (both sides in
      // registers), + the far tile edges
      const double Tk = plane_T(P, R, (double)k);
      double Fx[2][M], Fy[2][M];
      double cz[2][N];
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const double2* d = reinterpret_cast<const double2*>(D + (size_t)me[r] * D_NV + D_CZ);
        const double2 z01 = d[0], z23 = d[1];
        cz[r][0] = z01.x; cz[r][1] = z01.y; cz[r][2] = z23.x; cz[r][3] = z23.y;
      }
      FaceSide p, s;
#if PF_MU_TMEM
      // own sides from shared memory (the carried copy is in TMEM)
      (void)cz;
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        side_from_smem<L, NC>(D, me[r], D_CY, D_CZ, s);
        side_from_smem<L, NC>(D, me[r] - 1, D_CY, D_CZ, p);
        mu_face<L, TA>(P, Tk, p, s, Fx[r]);
      }
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        side_from_smem<L, NC>(D, me[r], D_CX, D_CZ, s);
        side_from_smem<L, NC>(D, r == 0 ? me[0] - HX : me[0], D_CX, D_CZ, p);
        mu_face<L, TA>(P, Tk, p, s, Fy[r]);
      }
#else
#pragma unroll
      for (int r = 0; r < 2; ++r) {
#pragma unroll
        for (int a = 0; a < N; ++a) {
          s.f[a] = Dp[r].f[a];
          s.c1[a] = Dp[r].c2[a];
          s.c2[a] = cz[r][a];
        }
#pragma unroll
        for (int u = 0; u < NSOL; ++u) s.ds[u] = Dp[r].ds[u];
        s.m[0] = Dp[r].m[0];
        s.m[1] = Dp[r].m[1];
        side_from_smem<L, NC>(D, me[r] - 1, D_CY, D_CZ, p);
        mu_face<L, TA>(P, Tk, p, s, Fx[r]);
      }
#pragma unroll
      for (int r = 0; r < 2; ++r) {
#pragma unroll
        for (int a = 0; a < N; ++a) {
          s.f[a] = Dp[r].f[a];
          s.c1[a] = Dp[r].c1[a];
          s.c2[a] = cz[r][a];
        }
#pragma unroll
        for (int u = 0; u < NSOL; ++u) s.ds[u] = Dp[r].ds[u];
        s.m[0] = Dp[r].m[0];
        s.m[1] = Dp[r].m[1];
        if (r == 0) {
          side_from_smem<L, NC>(D, me[0] - HX, D_CX, D_CZ, p);
        } else {  // the lower own cell, tangential x / z
#pragma unroll
          for (int a = 0; a < N; ++a) {
            p.f[a] = Dp[0].f[a];
            p.c1[a] = Dp[0].c1[a];
            p.c2[a] = cz[0][a];
          }
#pragma unroll
          for (int u = 0; u < NSOL; ++u) p.ds[u] = Dp[0].ds[u];
          p.m[0] = Dp[0].m[0];
          p.m[1] = Dp[0].m[1];
        }
        mu_face<L, TA>(P, Tk, p, s, Fy[r]);
      }
#endif
#pragma unroll
      for (int r = 0; r < 2; ++r)
#pragma unroll
        for (int i = 0; i < M; ++i) fxs[(i * MTY + 2 * w + r) * (MTX + 1) + lane] = Fx[r][i];
#pragma unroll
      for (int i = 0; i < M; ++i) fys[(i * (MTY + 1) + 2 * w) * MTX + lane] = Fy[0][i];
      if (w == 0) {  // +y face of the top tile edge, column `lane`
        double Fe[M];
        side_from_smem<L, NC>(D, hidx<MTX>(lane + 1, MTY), D_CX, D_CZ, p);
        side_from_smem<L, NC>(D, hidx<MTX>(lane + 1, MTY + 1), D_CX, D_CZ, s);
        mu_face<L, TA>(P, Tk, p, s, Fe);
#pragma unroll
        for (int i = 0; i < M; ++i) fys[(i * (MTY + 1) + MTY) * MTX + lane] = Fe[i];
      } else if (w == 1 && lane < MTY) {  // +x face of the right tile edge, row `lane`
        double Fe[M];
        side_from_smem<L, NC>(D, hidx<MTX>(MTX, lane + 1), D_CY, D_CZ, p);
        side_from_smem<L, NC>(D, hidx<MTX>(MTX + 1, lane + 1), D_CY, D_CZ, s);
        mu_face<L, TA>(P, Tk, p, s, Fe);
#pragma unroll
        for (int i = 0; i < M; ++i) fxs[(i * MTY + lane) * (MTX + 1) + MTX] = Fe[i];
      }
#if PF_MU_HASYNC
      cp_async_wait_all();  // this thread's staging copies, published by the barrier
#endif
      __syncthreads();
#pragma unroll
      for (int i = 0; i < M; ++i) {
        // lower row: its +y face is the upper row's -y face (registers)
        divxy[0][i] = (fxs[(i * MTY + 2 * w) * (MTX + 1) + lane + 1] - Fx[0][i]) + (Fy[1][i] - Fy[0][i]);
        divxy[1][i] = (fxs[(i * MTY + 2 * w + 1) * (MTX + 1) + lane + 1] - Fx[1][i]) +
                      (fys[(i * (MTY + 1) + 2 * w + 2) * MTX + lane] - Fy[1][i]);
      }
    }
  };
  for (int k = z0; k < z1; ++k) plane(BoolC<false>{}, k);
  plane(BoolC<true>{}, z1);
#if PF_MU_TMEM
  asm volatile("tcgen05.wait::st.sync.aligned;\n" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
  __syncthreads();
  if (w == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;\n" ::"r"(tm_base));
#endif
  };  // tile
#if PF_MU_PERS
  if (ts.skip == 2) {
    // persistent launch (tuning mu_pers): gridDim.x CTAs, each a balanced
    // contiguous share of the tile-planes in tile-major order, so that every
    // CTA slot of the GPU finishes at the same time (no partial last wave)
    // and a tile column restarts its z-march ~once instead of once per chunk.
    // The share's position lives in shared memory (volatile), not in
    // registers across the tile's march.
    __shared__ long long seg[2];
    const int ntx = (g.nx + MTX - 1) / MTX, nty = (g.ny + MTY - 1) / MTY;
    if (threadIdx.x == 0 && threadIdx.y == 0) {
      const i64 total = (i64)ntx * nty * g.nz;
      seg[0] = total * blockIdx.x / gridDim.x;
      seg[1] = total * (blockIdx.x + 1) / gridDim.x;
    }
    __syncthreads();
    volatile long long* vs = seg;
    for (;;) {
      const i64 lo = vs[0], hi = vs[1];
      if (lo >= hi) break;
      const i64 tl = lo / g.nz;
      const int z0 = (int)(lo - tl * g.nz);
      const int z1 = (int)min((i64)g.nz, (i64)z0 + (hi - lo));
      tile((int)(tl % ntx), (int)(tl / ntx), z0, z1);
      __syncthreads();  // every thread has read seg and finished the tile's shared-memory reads
      if (threadIdx.x == 0 && threadIdx.y == 0) vs[0] = lo + (z1 - z0);
      __syncthreads();
    }
    return;
  }
#endif
  const int tbx = blockIdx.x + ts.off[0], tby = blockIdx.y + ts.off[1], tbz = blockIdx.z + ts.off[2];
  if (ts.skip && tbx >= ts.lo[0] && tbx < ts.hi[0] && tby >= ts.lo[1] && tby < ts.hi[1] && tbz >= ts.lo[2] &&
      tbz < ts.hi[2])
    return;  // interior tile, done by the other launch
  tile(tbx, tby, tbz * ZC_MU, min(tbz * ZC_MU + ZC_MU, g.nz));
}

}  // namespace pf
