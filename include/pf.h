/*
 * pf.h -- C ABI of the B200-native grand-potential multiphase-field step.
 *
 * Implements the hot path of Bauer et al., "Code Generation for Massively
 * Parallel Phase-Field Simulations" (SC'19): one explicit time step of the
 * coupled phase-field (phi, N = 4 phases on the Gibbs simplex) and
 * chemical-potential (mu, K-1 = 2 components, with anti-trapping current)
 * equations on a 3-D Cartesian grid, as Algorithm 1 composes
 * them.  Citations "P:Lx-y" are lines of the paper text; "A<n>" are the
 * readings listed in DESIGN.md §3.
 *
 * Conventions for every entry point
 *   - Pure C99, no exceptions cross the ABI, no exit/abort.  Every call
 *     returns PF_OK (0) or a negative PF_E* status; pf_last_error() gives a
 *     human-readable message for the last failure on that context.
 *   - Field layout seen by callers: interior-only, structure of arrays,
 *     phi[alpha][z][y][x] and mu[i][z][y][x], x fastest, fp64, block-local.
 *   - Device buffers are OWNED BY THE CALLER (e.g. torch tensors) and sized
 *     by pf_query_layout(); the library never frees caller memory.  It owns
 *     only its NCCL communicator, streams, events and pinned scratch, released
 *     by pf_destroy().
 *   - All device work is enqueued on the caller's stream (pf_config.stream);
 *     calls are asynchronous unless documented as synchronous.  Errors of
 *     asynchronous work surface on a later call.
 *   - Multi-GPU: one process per GPU; world > 1 decomposes the global domain
 *     into procs[0] x procs[1] x procs[2] blocks, one per rank, with ghost
 *     layers exchanged by NCCL send/recv.  Calls marked
 *     "collective" must be made by every rank in the same order.
 */
#ifndef PF_H
#define PF_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ------------------------------------------------------ */
#define PF_OK 0
#define PF_EINVAL (-1)   /* invalid argument / configuration / parameters   */
#define PF_ENOMEM (-2)   /* buffer too small or allocation failed           */
#define PF_ECUDA (-3)    /* CUDA runtime error (incl. earlier async errors) */
#define PF_ENCCL (-4)    /* NCCL error or NCCL unavailable                  */
#define PF_ESTATE (-5)   /* wrong call order (e.g. step before init)        */
#define PF_ENUMERIC (-6) /* invariant monitor tripped (sum phi, phi >= 0)   */

/* ---- boundary conditions per side (reading A15) ------------------------ */
#define PF_BC_PERIODIC 0
#define PF_BC_NEUMANN 1      /* phi and mu: ghost = adjacent interior value */
#define PF_BC_DIRICHLET_MU 2 /* phi Neumann; mu ghost = mu_inf             */

#define PF_HOST 0
#define PF_DEVICE 1
#define PF_PHI 1u
#define PF_MU 2u

#define PF_N 4 /* phases (P1: 3 solids + liquid)  */
#define PF_M 2 /* chemical potentials K-1 (3 components)        */

/* kernel schedule (pf_set_variant); all agree with the oracle to <= 1e-12 */
#define PF_VARIANT_TUNED 0 /* z-marching, face fluxes computed once; generic */
#define PF_VARIANT_NAIVE 1 /* one thread per cell, every face computed twice */
#define PF_VARIANT_JIT 2   /* default: the tuned kernels specialised at run time
                              (NVRTC) with the parameters and the block
                              geometry as compile-time constants */
#define PF_VARIANT_SPLIT 3 /* the paper's "split" kernels: a
                              staggered kernel stores every face flux in a
                              global array (12 doubles per cell for phi, 6 for
                              mu), a cell kernel reads them back; bitwise equal
                              to PF_VARIANT_NAIVE ("full").  The staggered
                              array (12 x field doubles, 1.9 GB at 256^3) is
                              allocated by the library on first use and freed
                              by pf_destroy -- the one buffer it owns.     */

typedef struct pf_ctx pf_ctx;

typedef struct {
  int n_phases;     /* must be PF_N                                          */
  int n_mu;         /* must be PF_M                                          */
  int liquid;       /* index l of the liquid phase, 0..3 (eq. 10)            */
  int global[3];    /* global interior extents nx, ny, nz                    */
  int procs[3];     /* rank grid; product must equal world                   */
  int bc_lo[3];     /* PF_BC_* of the low side of x, y, z                    */
  int bc_hi[3];     /* PF_BC_* of the high side; periodic must match low     */
  int rank, world;  /* this process' rank, number of ranks (= GPUs)          */
  unsigned char nccl_uid[128]; /* ncclUniqueId bytes from rank 0 (world > 1); or
                                  "PFLOCAL:<name>" (NUL-terminated): the `world`
                                  blocks live in this process (e.g. on one GPU),
                                  each driven by its own host thread, and the
                                  halo exchange / reductions use an in-process
                                  transport (device copies ordered by events,
                                  host barriers per group call) instead of NCCL;
                                  CUDA-graph steps are off.  Test harness for
                                  the multi-block path on one device.       */
  int device;       /* CUDA device ordinal                                   */
  void* stream;     /* cudaStream_t borrowed from the caller (0 = legacy)     */
  double* phi[2];   /* caller-owned device buffers, pf_layout.phi_bytes each */
  double* mu[2];    /* caller-owned device buffers, pf_layout.mu_bytes each  */
  void* workspace;  /* caller-owned device buffer, pf_layout.workspace_bytes */
} pf_config;

typedef struct {
  int local[3];           /* this rank's interior extents nx, ny, nz          */
  int offset[3];          /* global index of its first interior cell          */
  int64_t pitch;          /* doubles per padded row (>= x_off + nx + 2)       */
  int64_t plane;          /* z stride in doubles                              */
  int64_t field;          /* component stride in doubles                      */
  int64_t x_off;          /* row offset of interior x = 0 (128-B aligned)     */
  /* cell (x,y,z) of component c is at c*field + (z+2)*plane + (y+2)*pitch +
   * x_off + x: one ghost layer (index -1, n) inside a guard ring of 2.
   * Default, structure of arrays [c][z][y][x]: plane = pitch*(ny+4),
   * field = plane*(nz+4).  Environment PF_LAYOUT=il at pf_query_layout /
   * pf_create time: plane-interleaved [z][c][y][x], field = pitch*(ny+4)
   * (one padded x-y plane), plane = PF_N*field (mu keeps PF_N slots per
   * z-plane, PF_M of them used).  Only the library addresses the padded buffers;
   * pf_init_fields / pf_download use the packed interior layout.           */
  size_t phi_bytes;       /* one time level of phi: ((PF_N-1)*field + (nz+4)*plane)*8 + 256 */
  size_t mu_bytes;        /* one time level of mu:  ((PF_M-1)*field + (nz+4)*plane)*8 + 256 */
  size_t workspace_bytes; /* tables, pack buffers, reduction scratch          */
} pf_layout;

/* Model parameters (eqs. 3-10 with A_ab = 1, P1).  Plain-old-data, fp64. */
typedef struct {
  double dx, dt, eps;                  /* grid spacing, time step, interface width */
  double gamma[PF_N][PF_N];            /* gamma_ab, symmetric, eqs. 4-5            */
  double gamma3[PF_N][PF_N][PF_N];     /* gamma_abd, symmetric, eq. 5              */
  double tau[PF_N][PF_N];              /* tau_ab, symmetric            */
  double A0[PF_N][PF_M][PF_M], A1[PF_N][PF_M][PF_M]; /* psi_a = mu.A mu + B.mu + C, */
  double B0[PF_N][PF_M], B1[PF_N][PF_M];             /* A, B, C affine in T (eq. 6) */
  double C0[PF_N], C1[PF_N];
  double D[PF_N][PF_M][PF_M];          /* D_alpha of the mobility, eq. 9           */
  double T0, G, v;                     /* T = T0 + G (z dx - v t)  [A13]           */
  double mu_inf[PF_M];                 /* inflow / Dirichlet value of mu           */
  double window_frac;                  /* moving window threshold fraction [A16]   */
  int window_check;                    /* check every n steps; 0 = window off      */
  /* Fluctuation term xi of eq. 7 (RNG P:L669-676), reading B4:
   * xi_a = xi_amp * U_a, U_a in (-1, 1) from Philox4x32-10 with counter
   * (global x, y, z, step mod 2^32) and key (xi_seed, step / 2^32), added to
   * the right-hand side of the phi equation outside the Lagrange multiplier.
   * xi_amp = 0: off (reading A17).  xi_amp >= 0 and finite.                  */
  double xi_amp;
  uint32_t xi_seed;
  /* P2 parameterisation (n_phases = 3, n_mu = 1 in pf_config; SURVEY §8(f)
   * NEXT-4): the leading 3 x 3 / 3 x 1 blocks of the arrays
   * above are used, and the gradient energy of eq. 4 is anisotropic,
   * a = sum_{a<b} gamma_ab A_ab(R_ab q_ab)^2 |q_ab|^2 with the cubic
   * A(p) = 1 - delta_ab (3 - 4 sum_i p_i^4 / |p|^4) of reading B6
   * (aniso = 1; 0: A = 1).  aniso_delta symmetric, >= 0 and < 1/5 (A > 0);
   * aniso_R[a][b] orthonormal 3 x 3, row-major, R_ab = R_ba.  The P2 path
   * has no fluctuation term (xi_amp = 0).  Ignored for P1.               */
  int aniso;
  double aniso_delta[PF_N][PF_N];
  double aniso_R[PF_N][PF_N][3][3];
} pf_params;

typedef struct {
  int64_t step;  /* completed steps; t_n = step * dt         */
  int64_t z_off; /* moving-window offset along z, in cells   */
} pf_state;

/* Sizes of the buffers a caller must provide for this configuration.
 * Reads cfg->global/procs/rank only.  PF_EINVAL on a bad decomposition. */
int pf_query_layout(const pf_config* cfg, pf_layout* out);

/* Host-only: neighbour ranks of this rank's block per dimension (nb_lo,
 * nb_hi; -1 = physical boundary, periodic dimensions wrap, possibly onto the
 * rank itself).  The halo exchange of dimension d sends the hi face to nb_hi
 * and the lo face to nb_lo, then receives the lo ghost from nb_lo and the hi
 * ghost from nb_hi (x, then y, then z; earlier dimensions' ghosts included
 * so that edges travel).  Reads cfg->global/procs/rank/world/bc_lo.        */
int pf_query_neighbors(const pf_config* cfg, int nb_lo[3], int nb_hi[3]);

/* Validate cfg, bind the caller's buffers, create streams/events and (world > 1)
 * the NCCL communicator from cfg->nccl_uid.  Collective when world > 1.     */
int pf_create(const pf_config* cfg, pf_ctx** out);
int pf_destroy(pf_ctx* ctx);

/* Copy the parameters (eqs. 3-10) after validation: positive dx, dt, eps,
 * tau, gamma; symmetric gamma, gamma3, tau; negative-definite symmetric part
 * of A_a(T) over the domain's T range (so dc/dmu is SPD, reading A6); finite
 * values; dt below the explicit stability bound (PF_EINVAL otherwise).      */
int pf_set_params(pf_ctx* ctx, const pf_params* p);

/* Load block-local interior fields (layout above) from host (where = PF_HOST)
 * or device (PF_DEVICE) memory.  Checks |sum phi - 1| <= 1e-12 and phi >= 0
 * (PF_EINVAL otherwise), resets step = 0 and z_off = 0, fills ghost layers
 * (collective halo exchange).  Synchronous.                                 */
int pf_init_fields(pf_ctx* ctx, const double* phi, const double* mu, int where);

/* Enqueue nsteps full time steps (Algorithm 1: phi-sweep, phi ghosts,
 * mu-sweep, mu ghosts, swap) plus, every window_check steps,
 * the moving-window check (front height max-reduction, shift if needed;
 * this synchronises the stream once per check).  Collective.               */
int pf_step(pf_ctx* ctx, int64_t nsteps);

/* Debug entry (SURVEY C.7 split diagnosis): one phi-sweep + phi ghosts, mu
 * copied unchanged, swap, step += 1.  Collective.                          */
int pf_step_phi_only(pf_ctx* ctx);

/* Refill ghost layers of the current fields: mask = PF_PHI | PF_MU.  Collective. */
int pf_halo_exchange(pf_ctx* ctx, unsigned mask);

/* Shift the current fields by k >= 0 planes along z (growth axis): new(z) =
 * old(z + k), the top k planes become liquid (phi = e_l, mu = mu_inf);
 * z_off += k (reading A16).  Requires procs[2] == 1.  Collective.          */
int pf_shift_window(pf_ctx* ctx, int k);

/* Front height H = max{z : exists (x,y) with phi_l < 1/2} over the global
 * domain, -1 if there is no solid.  Collective, synchronous. */
int pf_front_height(pf_ctx* ctx, int* H);

/* Invariant monitors of the current fields: out[0] = max |sum_a phi_a - 1|
 * (+inf if any phi or mu value is not finite), out[1] = min_a,cells phi_a
 * (global over ranks).  Collective, synchronous.                          */
int pf_monitor(pf_ctx* ctx, double out[2]);

/* Monitors inside pf_step (SURVEY §8(b) PF_ENUMERIC): every > 0 runs
 * pf_monitor at the end of every run of steps that reaches a multiple of
 * `every` (a run = one step, or one CUDA-graph replay of up to
 * window_check steps) and makes pf_step return PF_ENUMERIC -- the state
 * being the one after that run, pf_last_error naming the step and the
 * values -- when max|sum phi - 1| > tol, min phi < -tol, or a value is not
 * finite.  every = 0 (the default) turns them off.  tol >= 0.  Collective
 * when world > 1 (every rank takes the same decision).                    */
int pf_set_monitors(pf_ctx* ctx, int every, double tol);

/* Copy the current interior fields to host (where = PF_HOST) or device
 * (PF_DEVICE) memory in the layout above.  Synchronous.                     */
int pf_download(pf_ctx* ctx, double* phi, double* mu, int where);

int pf_get_state(const pf_ctx* ctx, pf_state* out);
int pf_set_state(pf_ctx* ctx, const pf_state* s);

/* Kernel schedule selection (PF_VARIANT_*), for ablations and parity.  The
 * JIT variant compiles on the first step after pf_set_params (~2 s, cached
 * per process); PF_ECUDA with the NVRTC log if that fails.                 */
int pf_set_variant(pf_ctx* ctx, int variant);

/* Tuning of the run-time specialised kernels (PF_VARIANT_JIT): the
 * thread-to-cell mapping (tile shape, z-chunk), the occupancy requested from
 * the register allocator and schedule transformations of the two sweeps.
 * The paper's code generator exposes exactly these as tunables -- "an
 * auto-tuning mechanism can then test and optimize different mappings"
 * and register-usage transformations tuned "for each kernel"
 * (P:L808-865).  Every setting computes the same result (the arithmetic per
 * cell does not depend on it; tests/test_gpu_autotune.py checks bitwise
 * equality).  Ranges (PF_EINVAL outside them):                              */
typedef struct {
  int phi_ty;        /* phi-sweep tile height (width 32): 4, 8, 16                  */
  int phi_minb;      /* phi-sweep CTAs per SM requested from ptxas: 1..8            */
  int phi_zc;        /* phi-sweep planes per CTA along z: 4..512                    */
  int phi_faces6;    /* 1: every thread computes all six faces of its cell (no
                        barrier); 0: each face once, +x/+y exchanged on chip        */
  int phi_unroll;    /* phi-sweep z-loop unroll factor: 1..4                        */
  int phi_prefetch;  /* software prefetch of the own column: 0 off, 1 L2, 2 L1      */
  int phi_pfd;       /* prefetch distance in planes: 1..4                           */
  int phi_xsh;       /* 1 (needs phi_faces6): the +x face flux comes from the next
                        lane by a warp shuffle, 31 cells per 32-lane tile row      */
  int phi_zrec;      /* 1: the -z face flux is recomputed per plane instead of
                        carried in registers (fewer registers, more fp64 work)   */
  int phi_xghost;    /* 1: the phi-sweep writes phi_dst's x ghost columns itself when
                        x is periodic inside the block (the ghost fill skips them) */
  int mu_ty;         /* mu-sweep tile height: 3..8 (tile width 32), 4..8 (width 16) */
  int mu_tx;         /* mu-sweep tile width: 16 or 32                               */
  int mu_minb;       /* mu-sweep CTAs per SM requested from ptxas: 1..6             */
  int mu_zc;         /* mu-sweep planes per CTA along z: 4..512                     */
  int mu_prefetch;   /* software prefetch of the own column: 0 off, 1 L2, 2 L1      */
  int mu_pfd;        /* prefetch distance in planes: 2..6                           */
  int mu_rpf;        /* 1: own cell's L1-missing loads one plane ahead in registers */
  int mu_halo_l1;    /* 1: halo-ring cells' next-plane lines prefetched into L1 (default 0 with mu_hasync, else 1) */
  int mu_fxreg;      /* 1: own -x/-y fluxes taken from registers in the divergence  */
  int mu_qreg;       /* 1: own cell's face-side data kept in registers from the
                        build (no shared-memory re-read; needs registers)        */
  int mu_ldhint;     /* L1 policy of the mu-sweep's phi_dst / mu loads: 0 default,
                        1 evict_first, 2 no_allocate, 3 no_allocate and the
                        two-rows sweep's own phi_src(k+2) loads evict_last        */
  int mu_hpipe;      /* 1: halo-ring cells' loads for plane k+1 issued at the end of
                        plane k's face phase (software pipelining)               */
  int mu_cly;        /* mu-sweep thread-block clusters of 1, 2 or 4 tiles stacked in
                        y (mu_tx = 32): tiles of a cluster march z in lockstep and
                        take the sides of a shared tile edge from each other's
                        shared memory instead of building a y-halo row            */
  int mu_rot;        /* 1: the tile rows and their per-plane roles (halo rows, edge
                        faces) rotated over the CTA's warps by a hash of the tile,
                        spreading them over the SM sub-partitions (mu_tx = 32)    */
  int mu_rpt;        /* mu-sweep tile rows per thread: 1, or 2 (mu_tx = 32, mu_ty 6
                        or 8: a 32 x mu_ty tile on 32 x mu_ty/2 threads)          */
  int phi_rpt;       /* phi-sweep tile rows per thread: 1, or 2 (phi_faces6 = 1,
                        phi_xsh = 0, even phi_ty: 32 x phi_ty/2 threads)           */
  int mu_pers;       /* 1: full mu-sweep launches are persistent (one CTA per
                        resident slot, each a balanced contiguous share of the
                        tile-planes; no partial last wave, one z-march restart per
                        share instead of one per mu_zc chunk); mu_rpt = 2 only     */
  int phi_pers;      /* 1: the same for the phi-sweep (phi_faces6 = 1, phi_rpt = 1) */
  int sched;         /* step schedule (S§7 step 6): 0 = two full sweeps (phi, ghosts,
                        mu); 1 = z-slab pipeline: per slab of `slab` mu z-chunks the
                        phi-sweep of the slab (shifted up one plane), its x/y
                        ghosts, then the mu-sweep of the slab while its phi_dst is
                        still in L2; 2 = the same slabs with the mu slabs on a
                        second stream, each after its phi slab (an event), so
                        that mu slab s and phi slab s+1 run concurrently and share
                        the SMs.  Applies to the JIT variant with no exchanged
                        dimension and a non-periodic z (DS); otherwise sched 0     */
  int slab;          /* mu z-chunks per slab of sched = 1, 2 (1..16)              */
  int mu_tmem;       /* 1: the two-rows mu-sweep keeps the carried side of plane
                        k-1 in tensor memory (tcgen05.st / ld, 68 columns per
                        thread) instead of registers, and re-reads the own
                        sides of the x / y faces from shared memory             */
  int mu_hcar;       /* 1: the two-rows mu-sweep carries the phi_src z column of
                        its halo ring in shared memory (a 3-plane ring): a halo
                        cell loads phi_src(k+1), the solids' phi_dst and mu per
                        plane (9 loads, not 26) and takes its tangential / z
                        differences from the ring; mu_rpt = 2, mu_hpipe = 0   */
  int mu_xshfl;      /* 1: the two-rows mu-sweep takes the x-neighbours' phi_src
                        of its own cells from the neighbour lanes' carried
                        values (warp shuffles; lanes 0 / 31 load the halo
                        column) instead of two L1 loads; mu_rpt = 2, mu_rpf = 1 */
  /* P2 parameterisation (pf_p2.cu; tuned by pf_autotune on a P2 context)  */
  int p2_phi;        /* P2 phi kernel: 0 side-staged (face sides in shared
                        memory), 1 z-marching with global-memory face operands
                        (default), 2 one thread per cell (every face twice)   */
  int p2_mu;         /* P2 mu kernel: the same three (default 0)              */
  int p2_phi_ty;     /* side-staged P2 phi: tile height (4 or 8) and CTAs per  */
  int p2_phi_minb;   /*   SM: (8, 2) default, (8, 1), (4, 3..6)                */
  int p2_mu_ty;      /* side-staged P2 mu: the same, default (4, 4)            */
  int p2_mu_minb;
  int p2_phi_pd;     /* side-staged P2 phi / mu: L2 prefetch distance in planes */
  int p2_mu_pd;      /*   (0 = off, 1..4; default 2)                           */
  int mu_atskip;     /* 1: the specialised mu-sweep skips the anti-trapping
                        current (eq. 10) in a warp whose faces all have it
                        exactly 0 (pb_l = 0 or every pb_s = 0: bulk phases,
                        solid-solid boundaries); same results, data-dependent
                        time; off by default and not searched by pf_autotune
                        (the benchmark reports it separately)                  */
  int mu_hasync;     /* 1: the two-rows mu-sweep stages its halo ring one plane
                        ahead with asynchronous global -> shared copies
                        (cp.async: phi_src two planes ahead into a 3-plane
                        ring, the solids' phi_dst and mu one plane ahead), so
                        a halo cell builds its side from shared memory with no
                        global load on the critical path (1: the ring's
                        cells, 8-B copies; 2: the whole halo tile's phi_src
                        planes in 16-B pieces, so the own cells read phi_src
                        from shared memory too).  Default 1; ignored (0)
                        unless mu_rpt = 2 and mu_hcar = mu_hpipe = mu_tmem =
                        0; 2 without mu_rpf acts as 1                          */
  int p2_mu_hasync;  /* 1: the specialised side-staged P2 mu-sweep (32 x 4 tiles) stages its
                        halo ring one build ahead with cp.async (as mu_hasync
                        1; default); same bits                                 */
} pf_tuning;

/* The built-in defaults (the measured best at 256^3 on one B200,
 * profiles/README.md), each overridable by the PF_* environment variable
 * of the same knob (PF_PHI_TY, PF_MU_MINB, ...). No device needed.          */
int pf_tuning_default(pf_tuning* out);
/* Select the tuning of this context; the specialised kernels are rebuilt on
 * the next step (cached per process).  PF_EINVAL for a value out of range.  */
int pf_set_tuning(pf_ctx* ctx, const pf_tuning* t);
int pf_get_tuning(const pf_ctx* ctx, pf_tuning* out);
/* Range check of a tuning without a context or device: PF_OK, or PF_EINVAL
 * with the reason in log[0..logn).                                         */
int pf_tuning_check(const pf_tuning* t, char* log, int logn);

/* Auto-tuning (S§8(f) NEXT-2): starting from the current tuning, a
 * coordinate search over the knobs of the kernels in `mask` (PF_PHI: the
 * phi-sweep, PF_MU: the mu-sweep), at most `passes` sweeps over the knobs.
 * Per knob, all candidate values are compiled concurrently with NVRTC on
 * host threads, then each candidate kernel is timed on this context's own
 * block and fields with CUDA events on the compute stream (median of `reps`
 * launches after 2 warm-up launches); a candidate replaces the current
 * setting if it is faster by more than 1 %.  With world > 1 the times are
 * max-reduced over ranks (NCCL) so that every rank selects the same tuning
 * (collective).  The timed launches read only the current time level and
 * write only the scratch level: the state (fields, step, z_off) is
 * unchanged.  Needs params and fields (PF_ESTATE otherwise) and the JIT
 * variant.  On return the context uses the best tuning found; `log` (may be
 * NULL) receives a JSON document with every candidate and its time,
 * truncated to logn bytes.  Synchronous.
 * Step level (mask has PF_PHI and PF_MU): the step schedules (two sweeps vs
 * the z-slab pipeline, tuning sched / slab) are timed as whole dry steps
 * (every kernel of a step, scratch level only, no swap) and the faster is
 * kept; with PF_AUTOTUNE_VARIANTS in `mask` the "full" (PF_VARIANT_NAIVE)
 * and "split" (PF_VARIANT_SPLIT, which allocates its staggered array) kernel
 * variants are timed the same way and reported ("variants" in the log); the
 * context keeps PF_VARIANT_JIT unless one of them is faster (S§8(f) NEXT-2:
 * full vs split vs fused).
 * P2 context (n_phases = 3): every kernel choice of each sweep in `mask`
 * (pf_tuning p2_*: side-staged / z-marching / one thread per cell, the
 * side-staged tile height x CTAs per SM and prefetch distance) is timed the
 * same way (median of `reps` launches, max over ranks, >= 1 % to replace
 * the current choice); `passes` and PF_AUTOTUNE_VARIANTS are ignored.      */
#define PF_AUTOTUNE_VARIANTS 4u
int pf_autotune(pf_ctx* ctx, unsigned mask, int passes, int reps, char* log, int logn);

/* Optional per-kernel timing with CUDA events on the compute stream:
 * pf_profile(ctx, 1) resets the counters and enables event timing
 * (pf_profile(ctx, 0) resets and disables it); pf_profile_read() returns the
 * accumulated milliseconds (0 if timing is disabled) and the number of
 * kernels launched since the reset, per category: phi-sweep (k = 0),
 * mu-sweep (1), ghost / halo pack-unpack (2), tables + window (3).
 * Synchronous read.                                                        */
int pf_profile(pf_ctx* ctx, int enable);
int pf_profile_read(pf_ctx* ctx, double ms[4], int64_t launches[4]);

/* Rank 0 of a world > 1 job: create the NCCL unique id (128 bytes) that the
 * caller broadcasts (e.g. with torch.distributed) into every rank's
 * pf_config.nccl_uid before pf_create.  PF_ENCCL if NCCL cannot be loaded. */
int pf_nccl_unique_id(unsigned char out[128]);

/* Build check without a device: compile the run-time specialised kernels
 * (PF_VARIANT_JIT) for parameters p, liquid index `liquid`, an n^3 block and
 * tuning t (NULL = pf_tuning_default) with NVRTC; optionally write the
 * sm_100a cubins to cubin_path (mu-sweep) and cubin_path + ".phi" (phi-sweep).
 * Returns the total cubin size in bytes, or -1 with the compiler log in
 * log[0..logn).                                                            */
int pf_jit_compile_only(const pf_params* p, int liquid, int n, const pf_tuning* t, const char* cubin_path, char* log,
                        int logn);
/* The same for the P2 sweeps (n_phases = 3, n_mu = 1; pf_p2 kernels on the
 * parameters p as compile-time constants): the phi- and mu-sweep of the
 * kernel choice in t (p2_* fields; NULL = default) for an n^3 block; cubins to cubin_path
 * (mu) and cubin_path + ".phi".  Returns the total size or -1 (log).     */
int pf_jit_compile_only_p2(const pf_params* p, int liquid, int n, const pf_tuning* t, const char* cubin_path, char* log,
                           int logn);

const char* pf_last_error(const pf_ctx* ctx);
const char* pf_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PF_H */
