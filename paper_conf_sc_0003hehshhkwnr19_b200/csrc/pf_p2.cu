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
#include <string.h>

#include <string>

#include "pf_internal.h"
#include "pf_p2_dev.cuh"

namespace pf {
namespace p2 {

// generic (ahead-of-time) kernels: the bodies of pf_p2_dev.cuh on the
// run-time parameter struct; the specialised build (pf_jit.cu, the default
// variant) instantiates the same bodies on compile-time constants
__global__ void __launch_bounds__(256) k_phi(Params P, Geom g, const double* __restrict__ ps,
                                             const double* __restrict__ ms, double* __restrict__ pd) {
  phi_naive_body(P, g, ps, ms, pd);
}
template <int L>
__global__ void __launch_bounds__(256) k_mu(Params P, Geom g, const double* __restrict__ ps,
                                            const double* __restrict__ pd, const double* __restrict__ ms,
                                            double* __restrict__ md) {
  mu_naive_body<Params, L>(P, g, ps, pd, ms, md);
}
// MB: CTAs per SM the kernel is compiled for (register cap 65536 / (128 MB))
template <int MB>
__global__ void __launch_bounds__(TXP * TYP, MB) k_phi_march(Params P, Geom g, const double* __restrict__ ps,
                                                         const double* __restrict__ ms, double* __restrict__ pd) {
  phi_march_body(P, g, ps, ms, pd);
}
template <int L, int MB>
__global__ void __launch_bounds__(TXP * TYP, MB) k_mu_march(Params P, Geom g, const double* __restrict__ ps,
                                                        const double* __restrict__ pd, const double* __restrict__ ms,
                                                        double* __restrict__ md) {
  mu_march_body<Params, L>(P, g, ps, pd, ms, md);
}
template <int L, int TY, int MB>
__global__ void __launch_bounds__(TXP * TY, MB) k_mu_side(Params P, Geom g, const double* __restrict__ ps,
                                                         const double* __restrict__ pd,
                                                         const double* __restrict__ ms, double* __restrict__ md) {
  mu_side_body<Params, L, TY>(P, g, ps, pd, ms, md);
}
template <int TY, int MB>
__global__ void __launch_bounds__(TXP * TY, MB) k_phi_side(Params P, Geom g, const double* __restrict__ ps,
                                                          const double* __restrict__ ms, double* __restrict__ pd) {
  phi_side_body<Params, TY>(P, g, ps, ms, pd);
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

// ---------------------------------------------------------------------------
// run-time specialisation of the P2 sweeps (pf_jit.cu compiles and loads it):
// the parameters as compile-time constants (struct KP2, PT::kSpec = true) and
// one kernel pf_p2_jit instantiating the body the kernel choice selects, on
// the same launch geometry as the generic kernels
// ---------------------------------------------------------------------------
namespace {
void put_d(std::string& o, double v) {
  char b[40];
  snprintf(b, sizeof b, "%.17g", v);
  o += b;
  if (!strpbrk(b, ".eEn")) o += ".0";  // keep it a double literal
}
void put_sd(std::string& o, const char* name, double v) {
  o += "  static constexpr double ";
  o += name;
  o += " = ";
  put_d(o, v);
  o += ";\n";
}
// a flat array of n doubles printed with the C shape `dims` (e.g. "[3][3]")
void put_ad(std::string& o, const char* name, const char* dims, const double* v, int n, int row) {
  o += "  static constexpr double ";
  o += name;
  o += dims;
  o += " = {";
  for (int i = 0; i < n; ++i) {
    if (i) o += ", ";
    put_d(o, v[i]);
    if (row && (i + 1) % row == 0 && i + 1 < n) o += "\n     ";
  }
  o += "};\n";
}
}  // namespace

void p2_launch_dims(const P2Cfg& c, const Geom& g, dim3* grid, dim3* block) {
  if (c.kern == 2) {
    *block = dim3(32, 4, 2);
    *grid = dim3((g.nx + 31) / 32, (g.ny + 3) / 4, (g.nz + 1) / 2);
  } else if (c.kern == 0) {
    *block = dim3(p2::TXP, c.ty);
    *grid = dim3((g.nx + p2::TXP - 1) / p2::TXP, (g.ny + c.ty - 1) / c.ty, (g.nz + p2::ZCS - 1) / p2::ZCS);
  } else {
    *block = dim3(p2::TXP, p2::TYP);
    *grid = dim3((g.nx + p2::TXP - 1) / p2::TXP, (g.ny + p2::TYP - 1) / p2::TYP, (g.nz + p2::ZCP - 1) / p2::ZCP);
  }
}

std::string p2_specialised_source(const void* Pv, const Geom& g, const P2Cfg& c, int which) {
  const p2::Params& P = *reinterpret_cast<const p2::Params*>(Pv);
  std::string o = "// generated by pf_p2.cu: P2 parameters as compile-time constants\n";
  // (the ring's static shared memory fits the 48-KB static limit beside the
  // side arrays of 32 x 4 tiles only)
  if (which == P2_MU && c.kern == 0 && c.hasync && c.ty == 4) o += "#define PF_P2_HASYNC 1\n";
  o += "#include \"pf_p2_dev.cuh\"\nnamespace pf {\nnamespace p2 {\nstruct KP2 {\n  static constexpr bool kSpec = true;\n";
  put_sd(o, "dx", P.dx);
  put_sd(o, "dt", P.dt);
  put_sd(o, "eps", P.eps);
  put_sd(o, "inv_eps", P.inv_eps);
  put_sd(o, "inv_dx", P.inv_dx);
  put_sd(o, "inv_dt", P.inv_dt);
  put_sd(o, "dt_over_eps", P.dt_over_eps);
  put_sd(o, "at_c", P.at_c);
  put_sd(o, "dTdt", P.dTdt);
  put_sd(o, "Tdz", P.Tdz);
  put_ad(o, "g", "[3][3]", &P.g[0][0], 9, 3);
  put_ad(o, "og", "[3][3]", &P.og[0][0], 9, 3);
  put_sd(o, "g3", P.g3);
  put_ad(o, "tau", "[3][3]", &P.tau[0][0], 9, 3);
  put_sd(o, "inv_tau_mean", P.inv_tau_mean);
  put_ad(o, "A0", "[3]", P.A0, 3, 0);
  put_ad(o, "A1", "[3]", P.A1, 3, 0);
  put_ad(o, "B0", "[3]", P.B0, 3, 0);
  put_ad(o, "B1", "[3]", P.B1, 3, 0);
  put_ad(o, "C0", "[3]", P.C0, 3, 0);
  put_ad(o, "C1", "[3]", P.C1, 3, 0);
  put_ad(o, "D", "[3]", P.D, 3, 0);
  put_ad(o, "delta", "[3][3]", &P.delta[0][0], 9, 3);
  put_ad(o, "R", "[3][3][9]", &P.R[0][0][0], 81, 9);
  put_sd(o, "mu_inf", P.mu_inf);
  char b[512];
  snprintf(b, sizeof b,
           "  static constexpr int liquid = %d, aniso = %d, prefetch = %d, side_pd = %d;\n"
           "  double Tbase;  // the only run-time value (per step)\n};\n}  // namespace p2\n",
           P.liquid, P.aniso, P.prefetch, c.pd);
  o += b;
  // the block geometry as compile-time constants (strides become immediates)
  snprintf(b, sizeof b,
           "struct KG {\n  static constexpr int nx = %d, ny = %d, nz = %d, z0 = %d, x0 = %d, y0 = %d, xwrap = 0;\n"
           "  static constexpr i64 pitch = %lldLL, plane = %lldLL, field = %lldLL, xoff = %lldLL;\n"
           "  __device__ __forceinline__ static constexpr i64 at(int x, int y, int z) {\n"
           "    return (i64)(z + GUARD) * plane + (i64)(y + GUARD) * pitch + xoff + x;\n  }\n};\n"
           "}  // namespace pf\nusing namespace pf;\nusing namespace pf::p2;\n",
           g.nx, g.ny, g.nz, g.z0, g.x0, g.y0, (long long)g.pitch, (long long)g.plane, (long long)g.field,
           (long long)g.xoff);
  o += b;
  const int L = P.liquid, mb = c.kern == 1 ? p2_minb() : c.mb;
  if (which == P2_PHI) {
    if (c.kern == 2)
      snprintf(b, sizeof b, "extern \"C\" __global__ void __launch_bounds__(256) pf_p2_jit(KP2 P, %s) {\n"
               "  phi_naive_body(P, KG{}, ps, ms, pd);\n}\n", "const double* __restrict__ ps, const double* __restrict__ ms, double* __restrict__ pd");
    else if (c.kern == 1)
      snprintf(b, sizeof b, "extern \"C\" __global__ void __launch_bounds__(TXP * TYP, %d) pf_p2_jit(KP2 P, %s) {\n"
               "  phi_march_body(P, KG{}, ps, ms, pd);\n}\n", mb, "const double* __restrict__ ps, const double* __restrict__ ms, double* __restrict__ pd");
    else
      snprintf(b, sizeof b, "extern \"C\" __global__ void __launch_bounds__(TXP * %d, %d) pf_p2_jit(KP2 P, %s) {\n"
               "  phi_side_body<KP2, %d>(P, KG{}, ps, ms, pd);\n}\n", c.ty, mb,
               "const double* __restrict__ ps, const double* __restrict__ ms, double* __restrict__ pd", c.ty);
  } else {
    const char* args = "const double* __restrict__ ps, const double* __restrict__ pd, const double* __restrict__ ms, "
                       "double* __restrict__ md";
    if (c.kern == 2)
      snprintf(b, sizeof b, "extern \"C\" __global__ void __launch_bounds__(256) pf_p2_jit(KP2 P, %s) {\n"
               "  mu_naive_body<KP2, %d>(P, KG{}, ps, pd, ms, md);\n}\n", args, L);
    else if (c.kern == 1)
      snprintf(b, sizeof b, "extern \"C\" __global__ void __launch_bounds__(TXP * TYP, %d) pf_p2_jit(KP2 P, %s) {\n"
               "  mu_march_body<KP2, %d>(P, KG{}, ps, pd, ms, md);\n}\n", mb, args, L);
    else
      snprintf(b, sizeof b, "extern \"C\" __global__ void __launch_bounds__(TXP * %d, %d) pf_p2_jit(KP2 P, %s) {\n"
               "  mu_side_body<KP2, %d, %d>(P, KG{}, ps, pd, ms, md);\n}\n", c.ty, mb, args, L, c.ty);
  }
  o += b;
  return o;
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
    else if (ty == 4 && mb == 5)
      p2::k_phi_side<4, 5><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
    else if (ty == 4 && mb == 6)
      p2::k_phi_side<4, 6><<<gr, b, 0, s>>>(P, g, ps, ms, pd);
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
   : ty == 4 && mb == 5 ? (p2::k_mu_side<LL, 4, 5><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md))   \
   : ty == 4 && mb == 6 ? (p2::k_mu_side<LL, 4, 6><<<gr, b, 0, s>>>(P, g, ps, pd, ms, md))   \
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

