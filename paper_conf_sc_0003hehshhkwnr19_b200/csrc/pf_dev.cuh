// pf_dev.cuh -- device-side types shared by the ahead-of-time (nvcc) build
// and the run-time specialised (NVRTC) build of the sweep kernels.  Must
// stay free of host headers: NVRTC compiles it as-is.
#pragma once

namespace pf {

typedef long long i64;

constexpr int N = 4;  // phases (P1: 3 solids + liquid)
constexpr int M = 2;  // chemical potentials, K - 1
constexpr int NSOL = N - 1;

// One ghost layer (indices -1 and n) inside an allocated guard ring of width
// 2 in y and z (and >= 2 in x), so that kernels may read any index in
// [-2, n+1] without bounds checks (edge threads of ragged tiles clamp to the
// ghost cell).
constexpr int GUARD = 2;

// Geometry of one block in the padded ghosted layout (pf_layout), run-time
// values.  The specialised build uses a type with the same members as
// compile-time constants.
struct Geom {
  int nx, ny, nz;
  int z0;  // global z index of local interior plane 0
  i64 pitch, plane, field, xoff;
  int x0, y0;  // global x / y index of local interior cell 0 (fluctuation counters)
  // x periodic within this block (x not exchanged): the tuned phi-sweep
  // writes the x ghost columns of phi_dst itself (store_x_ghost) and the
  // ghost fill skips them (S§8(a) a6: the strided columns are its costly part)
  int xwrap;
  __host__ __device__ __forceinline__ i64 at(int x, int y, int z) const {
    return (i64)(z + GUARD) * plane + (i64)(y + GUARD) * pitch + xoff + x;
  }
};

// x ghost columns of phi_dst written by the phi-sweep itself (x periodic
// inside the block): cell x = nx-1 is the ghost x = -1, cell 0 the ghost
// x = nx.  With nx % 4 == 0 the whole 32-B sector around the ghost is stored
// (x = -4..-1, nx..nx+3; the other slots are guard cells no result reads),
// so that L2 never merges a partial sector with DRAM.
template <class GT>
__device__ __forceinline__ void store_x_ghost(const GT& g, double* __restrict__ pd, int x, int y, int z, int a,
                                              double v) {
  if (!g.xwrap) return;
  const bool vec = (g.nx % 4) == 0;
  if (x == g.nx - 1) {
    double* q = pd + a * g.field + g.at(vec ? -4 : -1, y, z);
    if (vec) {
      reinterpret_cast<double2*>(q)[0] = make_double2(v, v);
      reinterpret_cast<double2*>(q)[1] = make_double2(v, v);
    } else {
      *q = v;
    }
  }
  if (x == 0) {
    double* q = pd + a * g.field + g.at(g.nx, y, z);
    if (vec) {
      reinterpret_cast<double2*>(q)[0] = make_double2(v, v);
      reinterpret_cast<double2*>(q)[1] = make_double2(v, v);
    } else {
      *q = v;
    }
  }
}

// Per-step values (T base of the frozen temperature, step index) of one step
// of a captured CUDA graph (pf_step, graph mode); the sweep bodies read
// R.Tbase and R.step of whatever R they get (DevParams or this).
struct StepVals {
  double Tbase;
  unsigned long long step;
};

// Tile selection of a sweep launch (interior / shell split for overlapping
// the halo exchange): tile = blockIdx + off; if skip, tiles
// with lo <= tile < hi in all three dimensions return at once.
struct TileSel {
  int off[3];
  int lo[3], hi[3];
  int skip;  // 1: skip the tiles inside [lo, hi); 2: persistent launch over all tiles (mu_pers)
};

// Scalars and coefficients of the model.  Passed by value to every kernel
// (kernel-parameter constant bank) in the generic build; folded into the
// code as compile-time constants in the specialised build.  T-dependent
// coefficients are stored as value = c0 + T c1 (eq. 6: A, B, C affine in T).
struct DevParams {
  double dx, dt, eps;
  double inv_dt;
  double inv_dx2;       // 1 / dx^2
  double phi_grad_c;    // eps / dx^2
  double inv_eps;
  double dt_over_eps;
  double at_c;          // 4 dx pi eps / (8 dt): anti-trapping prefactor in the units of mu_face
  double dTdt;          // -G v
  double Tbase, Tdz;    // T(local plane k) = Tbase + Tdz k; Tbase is set per step  [A13]
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
  double P0[N][4], P1[N][4];       // D_a chi_a / 2 (row-major 00 01 10 11), eq. 9 [A7]; /2: face sums
  double dchi0[NSOL][3], dchi1[NSOL][3];  // (chi_l - chi_s) / 2 (face sums of mu)
  double dB0[NSOL][M], dB1[NSOL][M];      // B_l - B_s
  double dcT[N][5];     // dc_a/dT = -(A1 + A1^T) mu - B1: [s00, s01, s11, -B1_0, -B1_1]
  int liquid;
  int TA;               // A1 != 0: chi and the mobility depend on T
  // fluctuation term (eq. 7) [B4]; per-step: step
  double xi_amp;        // 0 = off
  unsigned int xi_seed;
  unsigned long long step;  // time step n of the launch (Philox counter / key)
};

// Compile-time structure of a parameter set, known only to the specialised
// build (pf_jit.cu specialises it for its constant struct): all gamma_ab
// (a != b) equal, all gamma_abd equal.  The generic build keeps the general
// expressions (the paper's "generic application ... would have to spend
// FLOPs").
template <class PT>
struct ParamShape {
  static constexpr bool guni = false;   // gamma_ab uniform
  static constexpr bool g3uni = false;  // gamma_abd uniform
  static constexpr bool xi = true;      // fluctuation term compiled in (run-time amplitude, may be 0)
};

}  // namespace pf
