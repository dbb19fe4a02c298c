// pf_internal.h -- internal host-side declarations of the B200 phase-field
// library (not ABI).  Shared by the host runtime (pf_api.cu, pf_jit.cu) and
// the kernel translation units.  Nothing here is shared with the oracle
// (oracle/), by construction.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/pf.h"
#include "pf_dev.cuh"

static_assert(pf::N == PF_N && pf::M == PF_M, "ABI and device constants disagree");

namespace pf {

// ---- sweep launchers ---------------------------------------------------
void launch_phi_naive(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                      cudaStream_t s);
void launch_mu_naive(const DevParams& P, const Geom& g, const double* ps, const double* pd, const double* ms,
                     double* md, cudaStream_t s);
void launch_phi_tuned(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* pd,
                      cudaStream_t s);
// split variant: staggered fluxes through the global array J (12 x g.field doubles)
void launch_phi_split(const DevParams& P, const Geom& g, const double* ps, const double* ms, double* J, double* pd,
                      cudaStream_t s);
void launch_mu_split(const DevParams& P, const Geom& g, const double* ps, const double* pd, const double* ms,
                     double* J, double* md, cudaStream_t s);
// ts == nullptr: all tiles (grid ignored); else the selected tiles of `grid`
void launch_mu_tuned(const DevParams& P, const Geom& g, const TileSel* ts, dim3 grid, const double* ps,
                     const double* pd, const double* ms, double* md, cudaStream_t s);
// launch geometry of the tuned kernels (shared with the specialised build)
dim3 tuned_block();
dim3 tuned_block_mu(int mty, int mtx = 32);
dim3 tuned_grid_phi(const Geom& g, int pty, int zc = 0, int txc = 32);  // zc <= 0: the built-in z-chunk; txc: cells per row
dim3 tuned_block_phi(int pty);
dim3 tuned_grid_mu(const Geom& g, int mty, int zc = 0, int mtx = 32);
size_t tuned_mu_smem(int mty, int mtx = 32);  // mu-sweep tile: mtx x mty
int tuned_mu_ty_default();
size_t tuned_phi_smem();

// ---- ghost layers, halo exchange, window, reductions, copies ------------
// ghost fill of ncomp components; BC kind per side, -1 = filled by exchange
struct BCSpec {
  int kind_lo[3], kind_hi[3];
};
// skip_x: leave the x ghost columns (the sweeps wrap x, Geom::xwrap)
void launch_ghost_fill(const Geom& g, const BCSpec& bc, double* f, int ncomp, const double* dirichlet, cudaStream_t s,
                       bool skip_x = false);
void launch_ghost_stage(const Geom& g, int d, int klo, int khi, double* f, int ncomp, const double* dirichlet,
                        cudaStream_t s);
void launch_shift(const Geom& g, int k, int liquid, int nph, int nmu, const double* mu_inf, const double* phi_src,
                  const double* mu_src, double* phi_dst, double* mu_dst, cudaStream_t s);
void launch_front_height(const Geom& g, int liquid, const double* phi, int* out, cudaStream_t s);
void launch_monitor(const Geom& g, int nph, int nmu, const double* phi, const double* mu, unsigned long long* out2,
                    cudaStream_t s);
void launch_copy_interior(const Geom& g, int ncomp, const double* src, double* dst, int to_packed, cudaStream_t s);
// face pack/unpack for the ordered x -> y -> z halo exchange along dimension
// d: slab at index idx of dimension d, extended (ghosted) ranges for the
// dimensions before d so that edge ghosts travel.
size_t halo_slab_elems(const Geom& g, int d);
void launch_pack(const Geom& g, int d, int idx, int ncomp, const double* f, double* buf, cudaStream_t s);
void launch_unpack(const Geom& g, int d, int idx, int ncomp, double* f, const double* buf, cudaStream_t s);

void fill_dev_params(const pf_params& p, int liquid, DevParams* out);
bool plane_interleaved();  // field layout: [c][z][y][x] (default) or [z][c][y][x] (PF_LAYOUT=il)

// ---- P2 parameterisation (pf_p2.cu): 3 phases, 1 mu, anisotropic phi ----
size_t p2_params_size();                                                // bytes of the opaque parameter block
void p2_fill_params(const pf_params& p, int liquid, void* out);          // host values -> parameter block
// kernel choice of the P2 sweeps (pf_tuning p2_*)
struct P2Cfg {
  int kern;    // 0 side-staged, 1 z-marching, 2 one thread per cell
  int ty, mb;  // side-staged: tile height, CTAs per SM
  int pd;      // side-staged: L2 prefetch distance (planes)
  int hasync;  // side-staged mu, specialised build: halo ring staged by cp.async (p2_mu_hasync)
};
void p2_launch_phi(const void* P, const P2Cfg& c, double Tbase, const Geom& g, const double* ps, const double* ms,
                   double* pd, cudaStream_t s);
void p2_launch_mu(const void* P, const P2Cfg& c, double Tbase, const Geom& g, const double* ps, const double* pd,
                  const double* ms, double* md, cudaStream_t s);
// launch geometry of a kernel choice (the generic and the specialised kernels)
void p2_launch_dims(const P2Cfg& c, const Geom& g, dim3* grid, dim3* block);
// NVRTC source of the specialised P2 sweep `which` (P2_PHI / P2_MU) for kernel choice c
std::string p2_specialised_source(const void* P, const Geom& g, const P2Cfg& c, int which);

// ---- run-time specialisation (NVRTC) -------------------------------------
enum { JIT_PHI = 0, JIT_MU = 1, P2_PHI = 2, P2_MU = 3 };  // (P2_*: pf_tuning knobs of pf_p2.cu)
struct JitKernel;  // one specialised sweep compiled for (parameters, geometry, tuning)
void tuning_default(pf_tuning* t);            // built-in defaults + PF_* environment overrides
const char* tuning_check(const pf_tuning& t);  // nullptr if valid, else the reason
// build (or fetch from the process cache) a specialised kernel; returns
// nullptr and sets *err on failure
// owner: the pf_ctx the loaded module belongs to (one module per context and
// device; the compiled cubin itself is shared through a per-process cache)
JitKernel* jit_get(const void* owner, const DevParams& P, const Geom& g, const pf_tuning& t, int which,
                   std::string* err);
void jit_release(const void* owner);  // unload every module of `owner` (pf_destroy)
// compile the kernels of several tunings into the cubin cache, concurrently
// on up to nthreads host threads (no device needed)
void jit_precompile(const DevParams& P, const Geom& g, const std::vector<pf_tuning>& ts, int which, int nthreads);
// the same for already generated sources (P2: p2_specialised_source)
void jit_precompile_sources(const std::vector<std::string>& srcs, int nthreads);
// sv == nullptr: per-step values from P (by value); else a CUDA-graph step:
// they are copied from device memory sv into the module's constant first
// [zlo, zhi): a z-slab of planes (the slab schedule); zhi < 0 = all planes
cudaError_t jit_launch_phi(JitKernel* m, const DevParams& P, const double* ps, const double* ms, double* pd,
                           cudaStream_t s, const StepVals* sv = nullptr, int zlo = 0, int zhi = -1);
cudaError_t jit_launch_mu(JitKernel* m, const DevParams& P, const TileSel* ts, dim3 grid, const double* ps,
                          const double* pd, const double* ms, double* md, cudaStream_t s,
                          const StepVals* sv = nullptr);
// write the per-step values of the k steps of a graph launch (one block)
struct StepBatch {
  double Tbase[64];
  unsigned long long step0;
  int k;
};
void launch_set_steps(StepVals* dst, const StepBatch& b, cudaStream_t s);
// P2 (run-time specialised pf_p2_dev.cuh bodies): the kernel of choice c for
// parameter block P; launch with the per-step Tbase.  phi: (a, b, c) = (ps,
// ms, pd); mu: (a, b, c, d) = (ps, pd, ms, md)
JitKernel* jit_get_p2(const void* owner, const void* P, const Geom& g, const P2Cfg& c, int which, std::string* err);
cudaError_t jit_launch_p2(JitKernel* m, double Tbase, const double* a, const double* b, const void* c, double* d,
                          cudaStream_t s);
int jit_mu_ty_of(const JitKernel* m);
int jit_mu_tx_of(const JitKernel* m);
int jit_mu_zc_of(const JitKernel* m);
int phi_minb_for(int pty, int rpt);            // natural CTAs per SM of a tile shape
int mu_minb_for(int mty, int mtx, int rpt);

}  // namespace pf
