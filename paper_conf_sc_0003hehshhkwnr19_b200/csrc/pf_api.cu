// pf_api.cu -- host runtime and C ABI of the B200 phase-field step.
//
// Context management, padded layout, parameter validation and explicit
// stability bound, the per-step schedule of Algorithm 1 on
// the caller's stream, ghost layers / NCCL halo exchange, the
// moving window and the invariant monitors.  See include/pf.h for the ABI.
#include <dlfcn.h>
#include <math.h>
#include <nccl.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <array>
#include <condition_variable>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <type_traits>
#include <vector>

#include "pf_internal.h"
#include <nvtx3/nvToolsExt.h>  // header-only NVTX3: ranges for nsys / ncu timelines (no cost without a tool)

using namespace pf;

namespace {
// scoped NVTX range on the host thread around the enqueue of one phase of a
// step (phi-sweep, ghosts / exchange, mu-sweep, window); with a profiler
// attached the ranges line up with the kernels they enqueue
struct NvtxRange {
  explicit NvtxRange(const char* m) { nvtxRangePushA(m); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace


// ---------------------------------------------------------------------------
// NCCL, loaded on demand (dlopen) so that the library loads and runs without
// it for world == 1.  Prototypes from nccl.h.
// ---------------------------------------------------------------------------
namespace {
struct NcclApi {
  void* h = nullptr;
  decltype(&ncclCommInitRank) CommInitRank = nullptr;
  decltype(&ncclCommDestroy) CommDestroy = nullptr;
  decltype(&ncclSend) Send = nullptr;
  decltype(&ncclRecv) Recv = nullptr;
  decltype(&ncclGroupStart) GroupStart = nullptr;
  decltype(&ncclGroupEnd) GroupEnd = nullptr;
  decltype(&ncclAllReduce) AllReduce = nullptr;
  decltype(&ncclGetErrorString) GetErrorString = nullptr;
  decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
  bool load(std::string* err) {
    if (h) return true;
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* n : names) {
      h = dlopen(n, RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
      if (!h) h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
      if (h) break;
    }
    if (!h) {
      *err = std::string("cannot dlopen libnccl.so.2: ") + dlerror();
      return false;
    }
#define PF_SYM(field, name)                                   \
  field = reinterpret_cast<decltype(field)>(dlsym(h, name)); \
  if (!field) { *err = std::string("NCCL symbol missing: ") + name; return false; }
    PF_SYM(CommInitRank, "ncclCommInitRank");
    PF_SYM(CommDestroy, "ncclCommDestroy");
    PF_SYM(Send, "ncclSend");
    PF_SYM(Recv, "ncclRecv");
    PF_SYM(GroupStart, "ncclGroupStart");
    PF_SYM(GroupEnd, "ncclGroupEnd");
    PF_SYM(AllReduce, "ncclAllReduce");
    PF_SYM(GetErrorString, "ncclGetErrorString");
    PF_SYM(GetUniqueId, "ncclGetUniqueId");
#undef PF_SYM
    return true;
  }
};
NcclApi g_nccl;

// ---------------------------------------------------------------------------
// In-process transport (pf_config.nccl_uid = "PFLOCAL:<name>"): the `world`
// blocks of one decomposition live in one process, possibly on one device,
// each driven by its own host thread.  It replaces only the transport of
// the halo exchange (ncclSend / ncclRecv become device copies ordered by
// events) and of the max-reductions; the pack / unpack kernels, the ordered
// x -> y -> z stages, the interior / shell overlap and the window logic are
// the ones NCCL runs with.  Matching is NCCL's: per ordered pair of ranks the
// k-th send of a group call pairs with the k-th receive.  Used by the
// multi-block bitwise tests on one GPU (VERDICT r1 "next" 6); a test
// transport, not a data path.
// ---------------------------------------------------------------------------
struct LocalGroup {
  int world = 0;
  std::mutex m;
  std::condition_variable cv;
  int arrived = 0;
  unsigned long long gen = 0;
  std::vector<std::vector<std::deque<std::pair<const void*, size_t>>>> q;  // [src][dst] posted sends
  std::vector<cudaEvent_t> ready, done;                                   // per rank
  std::vector<std::vector<double>> red;                                   // per rank reduction inputs
  void barrier() {
    std::unique_lock<std::mutex> lk(m);
    const unsigned long long g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
};
std::mutex g_groups_mu;
std::map<std::string, std::weak_ptr<LocalGroup>> g_groups;

std::shared_ptr<LocalGroup> local_group(const std::string& name, int world) {
  std::lock_guard<std::mutex> lk(g_groups_mu);
  auto it = g_groups.find(name);
  if (it != g_groups.end())
    if (auto sp = it->second.lock()) return sp->world == world ? sp : nullptr;
  auto sp = std::make_shared<LocalGroup>();
  sp->world = world;
  sp->q.assign(world, std::vector<std::deque<std::pair<const void*, size_t>>>(world));
  sp->ready.assign(world, nullptr);
  sp->done.assign(world, nullptr);
  sp->red.assign(world, {});
  g_groups[name] = sp;
  return sp;
}

// one send / receive of a group call
struct XMsg {
  void* p;
  size_t bytes;
  int peer;
};
}  // namespace

// ---------------------------------------------------------------------------
struct pf_ctx {
  pf_config cfg;
  pf_layout lay;
  Geom g;
  int coord[3];           // rank coordinates in the rank grid
  int nb_lo[3], nb_hi[3];  // neighbour ranks (-1 = physical boundary)
  BCSpec bc_all;          // local BC kinds, -1 where a halo exchange fills the side
  bool exchange[3];       // dimension d is exchanged (procs[d] > 1 or forced)
  bool force_exchange = false;
  cudaStream_t stream = nullptr;
  double* phi[2];
  double* mu[2];
  int cur = 0;
  // workspace carve-up
  unsigned long long* red = nullptr;  // reduction scratch (4 x u64)
  double* sendbuf[3][2] = {};
  double* recvbuf[3][2] = {};
  // host
  unsigned long long* pinned = nullptr;
  pf_params hp;
  DevParams dp;
  bool have_params = false, have_fields = false;
  int64_t step = 0, z_off = 0;
  int variant = PF_VARIANT_JIT;
  // overlap of the halo exchange with interior work
  int first_ex = 3;                 // first exchanged dimension (3 = none)
  cudaStream_t comm_s = nullptr;    // exchange stream
  cudaStream_t mu_s = nullptr;      // sched = 2: the mu slabs, concurrent with the next phi slab
  std::vector<cudaEvent_t> ev_slab; // sched = 2: phi slab s (and its ghosts) done
  cudaEvent_t ev_slab_done = nullptr;
  cudaEvent_t ev_phi = nullptr, ev_phix = nullptr, ev_mu = nullptr, ev_mux = nullptr;
  bool mux_pending = false;         // mu exchange in flight on comm_s
  bool overlap = true;
  int64_t mu_launches_per_step = 1, ghost_launches_per_step = 0;  // launch accounting of graph replays
  JitKernel* jphi = nullptr;  // specialised sweeps for (dp, g, tune); reset by pf_set_params / pf_set_tuning
  JitKernel* jmu = nullptr;
  JitKernel* jp2[2] = {nullptr, nullptr};  // P2: specialised phi / mu sweeps and the kernel choices they hold
  P2Cfg jp2c[2] = {};
  pf_tuning tune;             // tuning of the specialised sweeps (pf_set_tuning, pf_autotune)
  // CUDA-graph steps (S§8(d) D.7): runs of steps between window checks are
  // captured once per (length, buffer parity) and replayed; the per-step
  // values (T base, step) are written to sv_dev before each replay and each
  // captured step copies its entry into the sweep modules' constant memory
  bool zero_copy_z = true;  // z exchanges send / receive whole planes in place (PF_ZC_EXCHANGE=0: pack)
  bool use_graph = true;
  int mon_every = 0;      // pf_set_monitors: check every n steps inside pf_step (0 = off)
  double mon_tol = 0.0;
  int64_t graph_min_cells = 128 * 128 * 128;  // PF_GRAPH=1: any size, PF_GRAPH=0: never
  cudaStream_t cap_s = nullptr;      // private stream the steps are captured on (the caller's may be legacy)
  StepVals* sv_dev = nullptr;        // [64] in the workspace
  const StepVals* cap_sv = nullptr;  // set while capturing one step of a graph
  typedef std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>> ProfPair;  // (category, start, end)
  std::vector<ProfPair> cap_prof;  // timing events recorded as graph nodes during a capture
  struct GraphEntry {
    int k, cur;
    cudaGraphExec_t exec;
    std::vector<ProfPair> prof;  // per-kernel timing events of the graph (pf_profile on)
    bool pending = false;        // replayed, times not yet collected
  };
  std::vector<GraphEntry> graphs;
  ncclComm_t comm = nullptr;
  std::shared_ptr<LocalGroup> lg;  // in-process transport instead of NCCL (world > 1, "PFLOCAL:")
  // P2 parameterisation (3 phases, 1 mu, anisotropic phi; pf_p2.cu)
  bool p2 = false;
  int nph = PF_N, nmu = PF_M;
  double* stag = nullptr;  // PF_VARIANT_SPLIT: staggered face fluxes (library-owned, freed by pf_destroy)
  std::vector<unsigned char> p2par;
  bool collective() const { return comm != nullptr || lg != nullptr; }
  // profiling
  bool prof = false;
  std::vector<cudaEvent_t> ev_pool;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> ev_open;
  double prof_ms[4] = {0, 0, 0, 0};
  int64_t prof_n[4] = {0, 0, 0, 0};
  int64_t nlaunch[4] = {0, 0, 0, 0};  // kernels launched per category since pf_profile()
  std::string err;
};

namespace {

void drop_graphs(pf_ctx* c) {
  for (auto& e : c->graphs) {
    if (e.pending && !e.prof.empty()) cudaEventSynchronize(e.prof.back().second.second);
    cudaGraphExecDestroy(e.exec);
    for (auto& pp : e.prof) {
      cudaEventDestroy(pp.second.first);
      cudaEventDestroy(pp.second.second);
    }
  }
  c->graphs.clear();
}

// per-kernel times of the last replay of a graph (its events are reused by
// the next replay): wait for it and add them up
void graph_prof_collect(pf_ctx* c, pf_ctx::GraphEntry& e) {
  if (!e.pending || e.prof.empty()) return;
  cudaEventSynchronize(e.prof.back().second.second);
  for (auto& pp : e.prof) {
    float ms = 0;
    cudaEventElapsedTime(&ms, pp.second.first, pp.second.second);
    c->prof_ms[pp.first] += ms;
    c->prof_n[pp.first] += 1;
  }
  e.pending = false;
}

int fail(pf_ctx* c, int code, const char* fmt, ...) {
  if (c) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    c->err = buf;
  }
  return code;
}

#define CU(call)                                                                          \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess) return fail(ctx, PF_ECUDA, "%s: %s", #call, cudaGetErrorString(e_)); \
  } while (0)

#define NC(call)                                                                                  \
  do {                                                                                            \
    ncclResult_t r_ = (call);                                                                     \
    if (r_ != ncclSuccess) return fail(ctx, PF_ENCCL, "%s: %s", #call, g_nccl.GetErrorString(r_)); \
  } while (0)

int check_launch(pf_ctx* ctx, const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ctx, PF_ECUDA, "%s launch: %s", what, cudaGetErrorString(e));
  return PF_OK;
}

size_t align256(size_t b) { return (b + 255) & ~(size_t)255; }

// One group of point-to-point messages on stream st (the transport of the
// halo exchange): NCCL grouped send / recv, or the in-process transport.
int xchg(pf_ctx* ctx, const std::vector<XMsg>& sends, const std::vector<XMsg>& recvs, cudaStream_t st) {
  if (ctx->comm) {
    NC(g_nccl.GroupStart());
    for (const XMsg& m : sends) NC(g_nccl.Send(m.p, m.bytes / sizeof(double), ncclDouble, m.peer, ctx->comm, st));
    for (const XMsg& m : recvs) NC(g_nccl.Recv(m.p, m.bytes / sizeof(double), ncclDouble, m.peer, ctx->comm, st));
    NC(g_nccl.GroupEnd());
    return PF_OK;
  }
  LocalGroup& G = *ctx->lg;
  const int me = ctx->cfg.rank;
  // 1. the send buffers are ready once the work enqueued so far is done
  CU(cudaEventRecord(G.ready[me], st));
  {
    std::lock_guard<std::mutex> lk(G.m);
    for (const XMsg& m : sends) G.q[me][m.peer].push_back({m.p, m.bytes});
  }
  G.barrier();
  // 2. each receive copies the matching send of its peer after the peer's event
  int rc = PF_OK;
  for (const XMsg& m : recvs) {
    std::pair<const void*, size_t> src(nullptr, 0);
    {
      std::lock_guard<std::mutex> lk(G.m);
      if (!G.q[m.peer][me].empty()) {
        src = G.q[m.peer][me].front();
        G.q[m.peer][me].pop_front();
      }
    }
    if (!src.first || src.second != m.bytes) {
      rc = fail(ctx, PF_ENCCL, "local transport: unmatched receive from rank %d (%zu bytes)", m.peer, m.bytes);
      continue;
    }
    cudaError_t e = cudaStreamWaitEvent(st, G.ready[m.peer], 0);
    if (e == cudaSuccess) e = cudaMemcpyAsync(m.p, src.first, m.bytes, cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) rc = fail(ctx, PF_ECUDA, "local transport copy: %s", cudaGetErrorString(e));
  }
  cudaEventRecord(G.done[me], st);
  G.barrier();
  // 3. a send buffer may be reused once its receivers have copied it
  for (const XMsg& m : sends) cudaStreamWaitEvent(st, G.done[m.peer], 0);
  G.barrier();  // nobody re-records its events before every wait above is enqueued
  return rc;
}

// max over ranks of n values in device memory (on ctx->stream), as u64 or f64
template <class T>
int allreduce_max(pf_ctx* ctx, T* dbuf, int n) {
  if (ctx->comm) {
    NC(g_nccl.AllReduce(dbuf, dbuf, n, std::is_same<T, double>::value ? ncclFloat64 : ncclUint64, ncclMax,
                        ctx->comm, ctx->stream));
    return PF_OK;
  }
  if (!ctx->lg) return PF_OK;
  LocalGroup& G = *ctx->lg;
  std::vector<T> v(n);
  CU(cudaStreamSynchronize(ctx->stream));
  CU(cudaMemcpy(v.data(), dbuf, n * sizeof(T), cudaMemcpyDeviceToHost));
  {
    std::lock_guard<std::mutex> lk(G.m);
    G.red[ctx->cfg.rank].assign(n, 0.0);
    memcpy(G.red[ctx->cfg.rank].data(), v.data(), n * sizeof(T));
  }
  G.barrier();
  {
    std::lock_guard<std::mutex> lk(G.m);
    for (int r = 0; r < G.world; ++r)
      for (int i = 0; i < n; ++i) {
        T x;
        memcpy(&x, &G.red[r][i], sizeof(T));
        if (x > v[i]) v[i] = x;
      }
  }
  G.barrier();
  CU(cudaMemcpy(dbuf, v.data(), n * sizeof(T), cudaMemcpyHostToDevice));
  return PF_OK;
}

void split(int n, int p, int r, int* len, int* off) {
  const int base = n / p, rem = n % p;
  *len = base + (r < rem ? 1 : 0);
  *off = r * base + std::min(r, rem);
}

}  // namespace
// Field layout in HBM: structure of arrays [c][z][y][x] by
// default; PF_LAYOUT=il selects the plane-interleaved [z][c][y][x] layout
// (every stencil load one base + immediate: -40 % integer instructions in
// the mu-sweep, but measured slower, phi 0.456 vs 0.421 ms at 256^3)
bool pf::plane_interleaved() {
  const char* e = getenv("PF_LAYOUT");
  return e && strcmp(e, "il") == 0;
}
namespace {

int layout_of(const pf_config* cfg, pf_layout* L, int coord[3]) {
  if (!cfg || !L) return PF_EINVAL;
  const int world = cfg->world < 1 ? 1 : cfg->world;
  int pr[3];
  for (int d = 0; d < 3; ++d) {
    pr[d] = cfg->procs[d] < 1 ? 1 : cfg->procs[d];
    if (cfg->global[d] < 1) return PF_EINVAL;
  }
  if (pr[0] * pr[1] * pr[2] != world || cfg->rank < 0 || cfg->rank >= world) return PF_EINVAL;
  int r = cfg->rank;
  coord[0] = r % pr[0];
  coord[1] = (r / pr[0]) % pr[1];
  coord[2] = r / (pr[0] * pr[1]);
  for (int d = 0; d < 3; ++d) {
    split(cfg->global[d], pr[d], coord[d], &L->local[d], &L->offset[d]);
    if (L->local[d] < 1) return PF_EINVAL;
  }
  const int nx = L->local[0], ny = L->local[1], nz = L->local[2];
  L->x_off = 16;  // interior x = 0 at a 128-B boundary; x in [-16, ...) addressable
  L->pitch = ((L->x_off + nx + GUARD) + 15) / 16 * 16;
  const int64_t pxy = L->pitch * (ny + 2 * GUARD);  // one padded x-y plane of one component
  if (plane_interleaved()) {
    // [z][c][y][x] (PF_LAYOUT=il): the components of a z-plane are adjacent
    // x-y planes (mu keeps PF_N slots per plane, two of them unused), so
    // every load of a cell's stencil -- all components, x/y/z neighbours --
    // is one base address plus an instruction immediate (< 8 MB)
    L->field = pxy;
    L->plane = (int64_t)PF_N * pxy;
  } else {
    // [c][z][y][x]: structure of arrays
    L->plane = pxy;
    L->field = pxy * (nz + 2 * GUARD);
  }
  const int64_t zspan = L->plane * (nz + 2 * GUARD);
  const int nph = cfg->n_phases == 3 ? 3 : PF_N, nmu = cfg->n_phases == 3 ? 1 : PF_M;  // P2: 3 phases, 1 mu
  L->phi_bytes = (size_t)((nph - 1) * L->field + zspan) * sizeof(double) + 256;  // +256: tail slack for vector loads
  L->mu_bytes = (size_t)((nmu - 1) * L->field + zspan) * sizeof(double) + 256;
  size_t ws = 256 + 1024;  // reduction scratch, per-step values of CUDA-graph steps
  Geom g{nx, ny, nz, L->offset[2], L->pitch, L->plane, L->field, L->x_off, L->offset[0], L->offset[1]};
  for (int d = 0; d < 3; ++d) ws += 4 * align256(halo_slab_elems(g, d) * PF_N * sizeof(double));
  L->workspace_bytes = ws;
  return PF_OK;
}

// Neighbour ranks of the block at rank-grid coordinates coord (-1 = physical
// boundary; periodic dimensions wrap, also onto the rank itself).
void neighbours_of(const pf_config* cfg, const int coord[3], int nb_lo[3], int nb_hi[3]) {
  int pr[3];
  for (int d = 0; d < 3; ++d) pr[d] = cfg->procs[d] < 1 ? 1 : cfg->procs[d];
  auto rank_of = [&](const int c[3]) { return c[0] + pr[0] * (c[1] + pr[1] * c[2]); };
  for (int d = 0; d < 3; ++d) {
    const bool periodic = cfg->bc_lo[d] == PF_BC_PERIODIC;
    int lo = coord[d] - 1, hi = coord[d] + 1;
    if (periodic) {
      lo = (lo + pr[d]) % pr[d];
      hi = hi % pr[d];
    }
    int cl[3] = {coord[0], coord[1], coord[2]}, ch[3] = {coord[0], coord[1], coord[2]};
    cl[d] = lo;
    ch[d] = hi;
    nb_lo[d] = (lo >= 0 && lo < pr[d]) ? rank_of(cl) : -1;
    nb_hi[d] = (hi >= 0 && hi < pr[d]) ? rank_of(ch) : -1;
  }
}

// Explicit (FTCS) stability bounds (SURVEY C.4 "dt"), in time units.
//  phi: linearised diffusivity of the gradient flux 2 sum_b gamma_ab phi_b^2 / tau <= 2 gamma_max / tau_min
//  mu:  D_eff = spectral radius of chi^{-1} M over sample points of the simplex
double eig2_max_abs(const double a[2][2]) {
  const double tr = a[0][0] + a[1][1], det = a[0][0] * a[1][1] - a[0][1] * a[1][0];
  const double disc = tr * tr / 4 - det;
  if (disc >= 0) return std::max(fabs(tr / 2 + sqrt(disc)), fabs(tr / 2 - sqrt(disc)));
  return sqrt(det > 0 ? det : -det);  // complex pair: |lambda| = sqrt(det)
}

double deff_at(const pf_params& p, const double* ph, double T) {
  double M[2][2] = {{0, 0}, {0, 0}}, X[2][2] = {{0, 0}, {0, 0}};
  for (int a = 0; a < PF_N; ++a) {
    double chi[2][2];
    for (int i = 0; i < 2; ++i)
      for (int j = 0; j < 2; ++j)
        chi[i][j] = -((p.A0[a][i][j] + p.A1[a][i][j] * T) + (p.A0[a][j][i] + p.A1[a][j][i] * T));
    const double x = ph[a], h = x * x * (3 - 2 * x);
    for (int i = 0; i < 2; ++i)
      for (int j = 0; j < 2; ++j) {
        X[i][j] += h * chi[i][j];
        M[i][j] += x * (p.D[a][i][0] * chi[0][j] + p.D[a][i][1] * chi[1][j]);
      }
  }
  const double det = X[0][0] * X[1][1] - X[0][1] * X[1][0];
  if (!(det > 0)) return INFINITY;
  const double inv[2][2] = {{X[1][1] / det, -X[0][1] / det}, {-X[1][0] / det, X[0][0] / det}};
  double K[2][2];
  for (int i = 0; i < 2; ++i)
    for (int j = 0; j < 2; ++j) K[i][j] = inv[i][0] * M[0][j] + inv[i][1] * M[1][j];
  return eig2_max_abs(K);
}

}  // namespace

namespace pf {
// device scalars and coefficients of pf_params (kernel-parameter constant
// bank of the generic build, compile-time constants of the specialised one)
void fill_dev_params(const pf_params& pr, int L, DevParams* out) {
  const pf_params* p = &pr;
  DevParams& D = *out;
  memset(&D, 0, sizeof D);
  D.dx = p->dx;
  D.dt = p->dt;
  D.eps = p->eps;
  D.inv_dt = 1.0 / p->dt;
  D.inv_dx2 = 1.0 / (p->dx * p->dx);
  D.phi_grad_c = p->eps / (p->dx * p->dx);
  D.inv_eps = 1.0 / p->eps;
  D.dt_over_eps = p->dt / p->eps;
  const double pi = 3.14159265358979323846;
  D.at_c = 4.0 * p->dx * pi * p->eps / (8.0 * p->dt);  // x 4: gradients scaled by 4 in mu_face
  D.dTdt = -p->G * p->v;
  D.Tdz = p->G * p->dx;
  D.mu_inf[0] = p->mu_inf[0];
  D.mu_inf[1] = p->mu_inf[1];
  for (int a = 0; a < PF_N; ++a)
    for (int b = 0; b < PF_N; ++b) {
      D.g[a][b] = a == b ? 0.0 : p->gamma[a][b];
      D.og[a][b] = a == b ? 0.0 : 16.0 / (pi * pi) * p->gamma[a][b];
    }
  const int others[4][3] = {{1, 2, 3}, {0, 2, 3}, {0, 1, 3}, {0, 1, 2}};
  for (int a = 0; a < PF_N; ++a) {
    const int* o = others[a];
    D.g3[a][0] = p->gamma3[a][o[0]][o[1]];
    D.g3[a][1] = p->gamma3[a][o[0]][o[2]];
    D.g3[a][2] = p->gamma3[a][o[1]][o[2]];
  }
  int k = 0;
  double tm = 0;
  for (int a = 0; a < PF_N; ++a)
    for (int b = a + 1; b < PF_N; ++b) {
      D.tau[k++] = p->tau[a][b];
      tm += p->tau[a][b];
    }
  D.inv_tau_mean = 6.0 / tm;
  bool ta = false;
  for (int a = 0; a < PF_N; ++a) {
    const double(*A0)[2] = p->A0[a];
    const double(*A1)[2] = p->A1[a];
    D.psiA[a][0] = A0[0][0];
    D.psiA[a][1] = A0[0][1] + A0[1][0];
    D.psiA[a][2] = A0[1][1];
    D.psiA1[a][0] = A1[0][0];
    D.psiA1[a][1] = A1[0][1] + A1[1][0];
    D.psiA1[a][2] = A1[1][1];
    for (int i = 0; i < 2; ++i) {
      D.B0[a][i] = p->B0[a][i];
      D.B1[a][i] = p->B1[a][i];
      for (int j = 0; j < 2; ++j) ta |= A1[i][j] != 0.0;
    }
    D.C0[a] = p->C0[a];
    D.C1[a] = p->C1[a];
    // chi = -(A + A^T)  [A6]
    D.chi0[a][0] = -(A0[0][0] + A0[0][0]);
    D.chi0[a][1] = -(A0[0][1] + A0[1][0]);
    D.chi0[a][2] = -(A0[1][1] + A0[1][1]);
    D.chi1[a][0] = -(A1[0][0] + A1[0][0]);
    D.chi1[a][1] = -(A1[0][1] + A1[1][0]);
    D.chi1[a][2] = -(A1[1][1] + A1[1][1]);
    // P = D_a chi_a (eq. 9, D left-multiplied [A7]), split in c0 + T c1
    const double X0[2][2] = {{D.chi0[a][0], D.chi0[a][1]}, {D.chi0[a][1], D.chi0[a][2]}};
    const double X1[2][2] = {{D.chi1[a][0], D.chi1[a][1]}, {D.chi1[a][1], D.chi1[a][2]}};
    for (int i = 0; i < 2; ++i)
      for (int j = 0; j < 2; ++j) {
        // x 1/2: the mu face uses face sums, not means
        D.P0[a][2 * i + j] = 0.5 * (p->D[a][i][0] * X0[0][j] + p->D[a][i][1] * X0[1][j]);
        D.P1[a][2 * i + j] = 0.5 * (p->D[a][i][0] * X1[0][j] + p->D[a][i][1] * X1[1][j]);
      }
    D.dcT[a][0] = D.chi1[a][0];
    D.dcT[a][1] = D.chi1[a][1];
    D.dcT[a][2] = D.chi1[a][2];
    D.dcT[a][3] = -p->B1[a][0];
    D.dcT[a][4] = -p->B1[a][1];
  }
  for (int s = 0; s < PF_N - 1; ++s) {
    const int a = s < L ? s : s + 1;
    for (int i = 0; i < 3; ++i) {
      D.dchi0[s][i] = 0.5 * (D.chi0[L][i] - D.chi0[a][i]);  // x 1/2: face sums of mu
      D.dchi1[s][i] = 0.5 * (D.chi1[L][i] - D.chi1[a][i]);
    }
    for (int i = 0; i < 2; ++i) {
      D.dB0[s][i] = p->B0[L][i] - p->B0[a][i];
      D.dB1[s][i] = p->B1[L][i] - p->B1[a][i];
    }
  }
  D.liquid = L;
  D.TA = ta ? 1 : 0;
  D.xi_amp = p->xi_amp;
  D.xi_seed = p->xi_seed;
}
}  // namespace pf

// ===========================================================================
extern "C" {

const char* pf_version(void) { return "pf-b200 0.1 (sm_100a, fp64)"; }

int pf_nccl_unique_id(unsigned char out[128]) {
  if (!out) return PF_EINVAL;
  std::string err;
  if (!g_nccl.load(&err)) return PF_ENCCL;
  ncclUniqueId id;
  if (g_nccl.GetUniqueId(&id) != ncclSuccess) return PF_ENCCL;
  memcpy(out, id.internal, 128);
  return PF_OK;
}

const char* pf_last_error(const pf_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

int pf_query_layout(const pf_config* cfg, pf_layout* out) {
  int coord[3];
  return layout_of(cfg, out, coord);
}

int pf_query_neighbors(const pf_config* cfg, int nb_lo[3], int nb_hi[3]) {
  pf_layout L;
  int coord[3];
  if (!nb_lo || !nb_hi) return PF_EINVAL;
  if (int r = layout_of(cfg, &L, coord)) return r;
  neighbours_of(cfg, coord, nb_lo, nb_hi);
  return PF_OK;
}

int pf_create(const pf_config* cfg, pf_ctx** out) {
  if (!cfg || !out) return PF_EINVAL;
  *out = nullptr;
  // P1 (4 phases, 2 mu) or P2 (3 phases, 1 mu)
  const bool is_p2 = cfg->n_phases == 3 && cfg->n_mu == 1;
  if (!((cfg->n_phases == PF_N && cfg->n_mu == PF_M) || is_p2) || cfg->liquid < 0 || cfg->liquid >= cfg->n_phases)
    return PF_EINVAL;
  pf_ctx* ctx = new (std::nothrow) pf_ctx();
  if (!ctx) return PF_ENOMEM;
  ctx->cfg = *cfg;
  ctx->p2 = is_p2;
  ctx->nph = is_p2 ? 3 : PF_N;
  ctx->nmu = is_p2 ? 1 : PF_M;
  tuning_default(&ctx->tune);
  if (layout_of(cfg, &ctx->lay, ctx->coord) != PF_OK) {
    delete ctx;
    return PF_EINVAL;
  }
  const pf_layout& L = ctx->lay;
  ctx->g = Geom{L.local[0], L.local[1], L.local[2], L.offset[2], L.pitch, L.plane, L.field, L.x_off,
                L.offset[0], L.offset[1]};
  for (int d = 0; d < 3; ++d) {
    const int blo = cfg->bc_lo[d], bhi = cfg->bc_hi[d];
    if (blo < 0 || blo > 2 || bhi < 0 || bhi > 2 || ((blo == PF_BC_PERIODIC) != (bhi == PF_BC_PERIODIC))) {
      delete ctx;
      return PF_EINVAL;
    }
  }
  for (int i = 0; i < 2; ++i) {
    ctx->phi[i] = cfg->phi[i];
    ctx->mu[i] = cfg->mu[i];
    if (!cfg->phi[i] || !cfg->mu[i]) {
      delete ctx;
      return PF_EINVAL;
    }
  }
  if (!cfg->workspace) {
    delete ctx;
    return PF_EINVAL;
  }
  ctx->stream = (cudaStream_t)cfg->stream;
  cudaError_t e = cudaSetDevice(cfg->device);
  if (e != cudaSuccess) {
    ctx->err = cudaGetErrorString(e);
    *out = ctx;
    return PF_ECUDA;
  }
  // workspace carve-up
  char* w = (char*)cfg->workspace;
  ctx->red = (unsigned long long*)w;
  w += 256;
  ctx->sv_dev = (StepVals*)w;
  w += 1024;
  for (int d = 0; d < 3; ++d) {
    const size_t b = align256(halo_slab_elems(ctx->g, d) * PF_N * sizeof(double));
    for (int s = 0; s < 2; ++s) {
      ctx->sendbuf[d][s] = (double*)w;
      w += b;
      ctx->recvbuf[d][s] = (double*)w;
      w += b;
    }
  }
  // neighbours and BC kinds
  const int world = cfg->world < 1 ? 1 : cfg->world;
  neighbours_of(cfg, ctx->coord, ctx->nb_lo, ctx->nb_hi);
  for (int d = 0; d < 3; ++d) {
    const int pr = cfg->procs[d] < 1 ? 1 : cfg->procs[d];
    ctx->exchange[d] = pr > 1;
    ctx->bc_all.kind_lo[d] = (ctx->exchange[d] && ctx->nb_lo[d] >= 0) ? -1 : cfg->bc_lo[d];
    ctx->bc_all.kind_hi[d] = (ctx->exchange[d] && ctx->nb_hi[d] >= 0) ? -1 : cfg->bc_hi[d];
  }
  if (world > 1 && memcmp(cfg->nccl_uid, "PFLOCAL:", 8) == 0) {
    // in-process transport (test harness: several blocks in one process)
    char name[121];
    memcpy(name, cfg->nccl_uid + 8, 120);
    name[120] = 0;
    ctx->lg = local_group(name, world);
    if (!ctx->lg || cfg->rank < 0 || cfg->rank >= world) {
      ctx->err = "local transport: group size mismatch or bad rank";
      *out = ctx;
      return PF_EINVAL;
    }
    cudaEvent_t er = nullptr, ed = nullptr;
    cudaError_t ee = cudaEventCreateWithFlags(&er, cudaEventDisableTiming);
    if (ee == cudaSuccess) ee = cudaEventCreateWithFlags(&ed, cudaEventDisableTiming);
    if (ee != cudaSuccess) {
      ctx->err = cudaGetErrorString(ee);
      *out = ctx;
      return PF_ECUDA;
    }
    std::lock_guard<std::mutex> lk(ctx->lg->m);
    ctx->lg->ready[cfg->rank] = er;
    ctx->lg->done[cfg->rank] = ed;
  } else if (world > 1) {
    if (!g_nccl.load(&ctx->err)) {
      *out = ctx;
      return PF_ENCCL;
    }
    ncclUniqueId id;
    static_assert(sizeof(id.internal) == 128, "ncclUniqueId size");
    memcpy(id.internal, cfg->nccl_uid, 128);
    ncclResult_t r = g_nccl.CommInitRank(&ctx->comm, world, id, cfg->rank);
    if (r != ncclSuccess) {
      ctx->err = std::string("ncclCommInitRank: ") + g_nccl.GetErrorString(r);
      *out = ctx;
      return PF_ENCCL;
    }
  }
  {
    // debug: periodic self-exchange through pack/unpack ("1": device copies;
    // "nccl": a 1-rank NCCL communicator, so that the NCCL send/recv and
    // all-reduce code of world > 1 runs on one GPU)
    const char* fe = getenv("PF_FORCE_EXCHANGE");
    const bool fnccl = fe && strcmp(fe, "nccl") == 0;
    ctx->force_exchange = fe && (fe[0] == '1' || fnccl);
    if (fnccl && world == 1) {
      if (!g_nccl.load(&ctx->err)) {
        *out = ctx;
        return PF_ENCCL;
      }
      ncclUniqueId id;
      ncclResult_t r = g_nccl.GetUniqueId(&id);
      if (r == ncclSuccess) r = g_nccl.CommInitRank(&ctx->comm, 1, id, 0);
      if (r != ncclSuccess) {
        ctx->err = std::string("1-rank NCCL communicator: ") + g_nccl.GetErrorString(r);
        *out = ctx;
        return PF_ENCCL;
      }
    }
  }
  // x periodic inside the block: the specialised phi-sweep may write phi_dst's x ghost columns
  ctx->g.xwrap = (cfg->bc_lo[0] == PF_BC_PERIODIC && !ctx->exchange[0] && !ctx->force_exchange) ? 1 : 0;
  if (getenv("PF_NO_XWRAP")) ctx->g.xwrap = 0;
  ctx->first_ex = 3;
  for (int d = 0; d < 3; ++d)
    if (ctx->exchange[d] || (ctx->force_exchange && cfg->bc_lo[d] == PF_BC_PERIODIC)) {
      ctx->first_ex = d;
      break;
    }
  {  // side stream: halo exchanges (N > 1) and the mu ghost fill (any N)
    const char* ov = getenv("PF_OVERLAP");
    ctx->overlap = !(ov && ov[0] == '0');
    const char* zc = getenv("PF_ZC_EXCHANGE");
    ctx->zero_copy_z = !(zc && zc[0] == '0');
    const char* gr = getenv("PF_GRAPH");
    ctx->use_graph = !(gr && gr[0] == '0') && !ctx->lg;  // the local transport syncs on the host: no graphs
    if (gr && gr[0] == '1') ctx->graph_min_cells = 0;
    e = cudaStreamCreateWithFlags(&ctx->comm_s, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&ctx->cap_s, cudaStreamNonBlocking);
    cudaEvent_t* evs[4] = {&ctx->ev_phi, &ctx->ev_phix, &ctx->ev_mu, &ctx->ev_mux};
    for (cudaEvent_t* ev : evs)
      if (e == cudaSuccess) e = cudaEventCreateWithFlags(ev, cudaEventDisableTiming);
    if (e != cudaSuccess) {
      ctx->err = cudaGetErrorString(e);
      *out = ctx;
      return PF_ECUDA;
    }
  }
  e = cudaMallocHost(&ctx->pinned, 64);
  if (e != cudaSuccess) {
    ctx->err = cudaGetErrorString(e);
    *out = ctx;
    return PF_ECUDA;
  }
  *out = ctx;
  return PF_OK;
}

int pf_destroy(pf_ctx* ctx) {
  if (!ctx) return PF_OK;
  if (ctx->stream || true) cudaStreamSynchronize(ctx->stream);
  for (auto ev : ctx->ev_pool) cudaEventDestroy(ev);
  for (auto& o : ctx->ev_open) {
    cudaEventDestroy(o.second.first);
    cudaEventDestroy(o.second.second);
  }
  drop_graphs(ctx);
  jit_release(ctx);
  if (ctx->stag) cudaFree(ctx->stag);
  if (ctx->comm) g_nccl.CommDestroy(ctx->comm);
  if (ctx->lg) {
    std::lock_guard<std::mutex> lk(ctx->lg->m);
    const int r = ctx->cfg.rank;
    if (ctx->lg->ready[r]) cudaEventDestroy(ctx->lg->ready[r]);
    if (ctx->lg->done[r]) cudaEventDestroy(ctx->lg->done[r]);
    ctx->lg->ready[r] = ctx->lg->done[r] = nullptr;
  }
  if (ctx->comm_s) {
    cudaStreamSynchronize(ctx->comm_s);
    cudaStreamDestroy(ctx->comm_s);
  }
  if (ctx->cap_s) cudaStreamDestroy(ctx->cap_s);
  if (ctx->mu_s) {
    cudaStreamSynchronize(ctx->mu_s);
    cudaStreamDestroy(ctx->mu_s);
  }
  for (cudaEvent_t ev : ctx->ev_slab) cudaEventDestroy(ev);
  if (ctx->ev_slab_done) cudaEventDestroy(ctx->ev_slab_done);
  for (cudaEvent_t ev : {ctx->ev_phi, ctx->ev_phix, ctx->ev_mu, ctx->ev_mux})
    if (ev) cudaEventDestroy(ev);
  if (ctx->pinned) cudaFreeHost(ctx->pinned);
  delete ctx;
  return PF_OK;
}

// ---------------------------------------------------------------------------
// P2 parameters (3 phases, 1 mu, anisotropic phi): validation, explicit
// stability bound, parameter block of pf_p2.cu
static int set_params_p2(pf_ctx* ctx, const pf_params* p) {
  const int L = ctx->cfg.liquid;
  auto finite = [](double v) { return isfinite(v); };
  const double* raw = (const double*)p;
  for (size_t i = 0; i < offsetof(pf_params, window_check) / sizeof(double); ++i)
    if (!finite(raw[i])) return fail(ctx, PF_EINVAL, "non-finite parameter at offset %zu", i);
  if (!(p->dx > 0 && p->dt > 0 && p->eps > 0)) return fail(ctx, PF_EINVAL, "dx, dt, eps must be > 0");
  if (p->xi_amp != 0.0) return fail(ctx, PF_EINVAL, "the P2 path has no fluctuation term (xi_amp = 0)");
  double gmax = 0, tmin = INFINITY, dmax = 0;
  for (int a = 0; a < 3; ++a)
    for (int b = 0; b < 3; ++b) {
      if (p->gamma[a][b] != p->gamma[b][a] || p->tau[a][b] != p->tau[b][a])
        return fail(ctx, PF_EINVAL, "gamma and tau must be symmetric");
      if (a == b) continue;
      if (!(p->gamma[a][b] > 0 && p->tau[a][b] > 0)) return fail(ctx, PF_EINVAL, "gamma_ab, tau_ab must be > 0");
      gmax = std::max(gmax, p->gamma[a][b]);
      tmin = std::min(tmin, p->tau[a][b]);
      if (p->aniso) {
        const double d = p->aniso_delta[a][b];
        if (!(d >= 0.0 && d < 0.2 && finite(d)) || d != p->aniso_delta[b][a])
          return fail(ctx, PF_EINVAL, "aniso_delta symmetric, 0 <= delta < 1/5");
        dmax = std::max(dmax, d);
        for (int i = 0; i < 3; ++i)
          for (int j = 0; j < 3; ++j) {
            double s = 0.0;
            for (int k = 0; k < 3; ++k) s += p->aniso_R[a][b][i][k] * p->aniso_R[a][b][j][k];
            if (!(fabs(s - (i == j ? 1.0 : 0.0)) < 1e-12) || p->aniso_R[a][b][i][j] != p->aniso_R[b][a][i][j])
              return fail(ctx, PF_EINVAL, "aniso_R[%d][%d] must be orthonormal and R_ab = R_ba", a, b);
          }
      }
    }
  double dmx = 0.0;
  const double Tlo = p->T0 - fabs(p->G) * (ctx->cfg.global[2] + 2) * p->dx, Thi = p->T0 + fabs(p->G) * (ctx->cfg.global[2] + 2) * p->dx;
  for (int a = 0; a < 3; ++a)
    for (double T : {Tlo, Thi}) {
      const double chi = -2.0 * (p->A0[a][0][0] + p->A1[a][0][0] * T);
      if (!(chi > 0)) return fail(ctx, PF_EINVAL, "A_%d(T=%g) must be < 0 (dc/dmu > 0)", a, T);
      dmx = std::max(dmx, p->D[a][0][0]);
      if (!(p->D[a][0][0] >= 0)) return fail(ctx, PF_EINVAL, "D_%d must be >= 0", a);
    }
  // phi: the gradient coefficient grows by up to (1 + delta)^2 and the
  // derivative terms of A; mu (M = 1): D_eff = sum_a g_a D_a chi_a / sum_a
  // h_a chi_a, sampled over the simplex (vertices, edge midpoints,
  // barycentre, 1000 seeded points) at the extreme temperatures
  const double dt_phi = tmin * p->dx * p->dx / (12.0 * gmax * (1.0 + dmax) * (1.0 + dmax) * (1.0 + 8.0 * dmax));
  std::vector<std::array<double, 3>> pts = {{1, 0, 0}, {0, 1, 0}, {0, 0, 1}, {0.5, 0.5, 0}, {0.5, 0, 0.5},
                                            {0, 0.5, 0.5}, {1.0 / 3, 1.0 / 3, 1.0 / 3}};
  uint64_t sd = 20191117ull;
  for (int i = 0; i < 1000; ++i) {
    std::array<double, 3> v;
    double sum = 0;
    for (int a = 0; a < 3; ++a) {
      sd = sd * 6364136223846793005ull + 1442695040888963407ull;
      v[a] = -log(((sd >> 11) + 0.5) * (1.0 / 9007199254740992.0));
      sum += v[a];
    }
    for (int a = 0; a < 3; ++a) v[a] /= sum;
    pts.push_back(v);
  }
  double deff = 0.0;
  for (const auto& v : pts)
    for (double T : {Tlo, Thi}) {
      double num = 0.0, den = 0.0;
      for (int a = 0; a < 3; ++a) {
        const double chi = -2.0 * (p->A0[a][0][0] + p->A1[a][0][0] * T);
        num += v[a] * p->D[a][0][0] * chi;
        den += v[a] * v[a] * (3.0 - 2.0 * v[a]) * chi;
      }
      deff = std::max(deff, num / den);
    }
  (void)dmx;
  const double dt_mu = deff > 0 ? p->dx * p->dx / (6.0 * deff) : INFINITY;
  if (p->dt > dt_phi || p->dt > dt_mu)
    return fail(ctx, PF_EINVAL, "dt = %g exceeds the explicit stability bound min(%g [phi], %g [mu])", p->dt, dt_phi,
                dt_mu);
  if (p->window_check < 0 || (p->window_check > 0 && !(p->window_frac > 0 && p->window_frac < 1)))
    return fail(ctx, PF_EINVAL, "window_check >= 0 and 0 < window_frac < 1");
  if (p->window_check > 0 && ctx->cfg.procs[2] != 1)
    return fail(ctx, PF_EINVAL, "the moving window needs the growth axis unsplit (procs[2] == 1)");
  ctx->p2par.assign(p2_params_size(), 0);
  p2_fill_params(*p, L, ctx->p2par.data());
  ctx->hp = *p;
  ctx->have_params = true;
  ctx->jphi = ctx->jmu = ctx->jp2[0] = ctx->jp2[1] = nullptr;
  drop_graphs(ctx);
  return PF_OK;
}

int pf_set_params(pf_ctx* ctx, const pf_params* p) {
  if (!ctx || !p) return PF_EINVAL;
  if (ctx->p2) return set_params_p2(ctx, p);
  const int L = ctx->cfg.liquid;
  auto finite = [](double v) { return isfinite(v); };
  const double* raw = (const double*)p;
  for (size_t i = 0; i < offsetof(pf_params, window_check) / sizeof(double); ++i)
    if (!finite(raw[i])) return fail(ctx, PF_EINVAL, "non-finite parameter at offset %zu", i);
  if (!(p->dx > 0 && p->dt > 0 && p->eps > 0)) return fail(ctx, PF_EINVAL, "dx, dt, eps must be > 0");
  double gmax = 0, tmin = INFINITY;
  for (int a = 0; a < PF_N; ++a)
    for (int b = 0; b < PF_N; ++b) {
      if (p->gamma[a][b] != p->gamma[b][a] || p->tau[a][b] != p->tau[b][a])
        return fail(ctx, PF_EINVAL, "gamma and tau must be symmetric");
      if (a == b) continue;
      if (!(p->gamma[a][b] > 0 && p->tau[a][b] > 0)) return fail(ctx, PF_EINVAL, "gamma_ab, tau_ab must be > 0");
      gmax = std::max(gmax, p->gamma[a][b]);
      tmin = std::min(tmin, p->tau[a][b]);
    }
  for (int a = 0; a < PF_N; ++a)
    for (int b = 0; b < PF_N; ++b)
      for (int d = 0; d < PF_N; ++d)
        if (p->gamma3[a][b][d] != p->gamma3[b][a][d] || p->gamma3[a][b][d] != p->gamma3[a][d][b])
          return fail(ctx, PF_EINVAL, "gamma3 must be symmetric");
  if (p->window_check < 0 || (p->window_check > 0 && !(p->window_frac > 0 && p->window_frac < 1)))
    return fail(ctx, PF_EINVAL, "window_check >= 0 and 0 < window_frac < 1");
  if (p->window_check > 0 && ctx->cfg.procs[2] != 1)  // checked here, not at the first shift
    return fail(ctx, PF_EINVAL, "the moving window needs the growth axis unsplit (procs[2] == 1)");
  if (!(std::isfinite(p->xi_amp) && p->xi_amp >= 0.0))
    return fail(ctx, PF_EINVAL, "xi_amp must be finite and >= 0");
  // T range over the global domain at t = 0 (frozen gradient; window keeps it bounded)
  const double zmax = (double)ctx->cfg.global[2];
  const double Ts[2] = {p->T0 - fabs(p->G) * p->dx, p->T0 + fabs(p->G) * (zmax + 1) * p->dx};
  for (double T : Ts)
    for (int a = 0; a < PF_N; ++a) {
      double c00 = -2 * (p->A0[a][0][0] + p->A1[a][0][0] * T), c11 = -2 * (p->A0[a][1][1] + p->A1[a][1][1] * T);
      double c01 = -((p->A0[a][0][1] + p->A1[a][0][1] * T) + (p->A0[a][1][0] + p->A1[a][1][0] * T));
      if (!(c00 > 0 && c00 * c11 - c01 * c01 > 0))
        return fail(ctx, PF_EINVAL, "A_%d(T=%g) is not negative definite (dc/dmu must be SPD)", a, T);
    }
  // stability bounds
  const double dt_phi = tmin * p->dx * p->dx / (12.0 * gmax);
  double deff = 0;
  {
    std::vector<std::vector<double>> pts;
    for (int a = 0; a < PF_N; ++a) {  // vertices, edge / face midpoints, barycentre
      std::vector<double> v(PF_N, 0.0);
      v[a] = 1;
      pts.push_back(v);
      for (int b = a + 1; b < PF_N; ++b) {
        std::vector<double> e(PF_N, 0.0);
        e[a] = e[b] = 0.5;
        pts.push_back(e);
        for (int c = b + 1; c < PF_N; ++c) {
          std::vector<double> f(PF_N, 0.0);
          f[a] = f[b] = f[c] = 1.0 / 3;
          pts.push_back(f);
        }
      }
    }
    pts.push_back(std::vector<double>(PF_N, 0.25));
    uint64_t s = 20191117ull;  // seeded random points on the simplex
    for (int i = 0; i < 1000; ++i) {
      std::vector<double> v(PF_N);
      double sum = 0;
      for (int a = 0; a < PF_N; ++a) {
        s = s * 6364136223846793005ull + 1442695040888963407ull;
        double u = ((s >> 11) + 0.5) * (1.0 / 9007199254740992.0);
        v[a] = -log(u);
        sum += v[a];
      }
      for (int a = 0; a < PF_N; ++a) v[a] /= sum;
      pts.push_back(v);
    }
    for (auto& v : pts)
      for (double T : Ts) deff = std::max(deff, deff_at(*p, v.data(), T));
  }
  const double dt_mu = deff > 0 ? p->dx * p->dx / (6.0 * deff) : INFINITY;
  if (p->dt > dt_phi || p->dt > dt_mu)
    return fail(ctx, PF_EINVAL, "dt = %g exceeds the explicit stability bound min(%g [phi], %g [mu])", p->dt, dt_phi,
                dt_mu);
  pf::fill_dev_params(*p, L, &ctx->dp);
  ctx->hp = *p;
  ctx->have_params = true;
  ctx->jphi = ctx->jmu = ctx->jp2[0] = ctx->jp2[1] = nullptr;
  drop_graphs(ctx);
  return PF_OK;
}

// ---------------------------------------------------------------------------
// ghost layers of one field set (Alg. 1 lines 2 / 4): local BCs + halo exchange
// ---------------------------------------------------------------------------
// dimensions [d0, d1) of the ordered x -> y -> z ghost fill, on stream `st`
// x_done: the producing sweep already wrote the x ghost columns (Geom::xwrap)
static int fill_ghost_dims(pf_ctx* ctx, double* f, int ncomp, bool is_mu, int d0, int d1, cudaStream_t st,
                           bool x_done = false) {
  NvtxRange nr(is_mu ? "pf mu ghosts / exchange" : "pf phi ghosts / exchange");
  const double* dir = is_mu ? ctx->hp.mu_inf : nullptr;
  const bool any_ex = ctx->first_ex < 3;
  const bool skipx = x_done;
  if (!any_ex && d0 == 0 && d1 == 3) {
    launch_ghost_fill(ctx->g, ctx->bc_all, f, ncomp, dir, st, skipx);
    ctx->nlaunch[2] += 1;
    return check_launch(ctx, "ghost_fill");
  }
  // ordered x -> y -> z stages so that edge ghosts travel with the slabs
  for (int d = d0; d < d1; ++d) {
    const bool ex = ctx->exchange[d] || (ctx->force_exchange && ctx->cfg.bc_lo[d] == PF_BC_PERIODIC);
    if (!ex) {
      if (d == 0 && skipx) continue;
      launch_ghost_stage(ctx->g, d, ctx->cfg.bc_lo[d], ctx->cfg.bc_hi[d], f, ncomp, dir, st);
      ctx->nlaunch[2] += 1;
      if (int r = check_launch(ctx, "ghost_stage")) return r;
      continue;
    }
    const int n = d == 0 ? ctx->g.nx : (d == 1 ? ctx->g.ny : ctx->g.nz);
    const size_t cnt = halo_slab_elems(ctx->g, d) * ncomp;
    const int lo = ctx->nb_lo[d] >= 0 ? ctx->nb_lo[d] : -1;
    const int hi = ctx->nb_hi[d] >= 0 ? ctx->nb_hi[d] : -1;
    if (d == 2 && ctx->collective() && ctx->zero_copy_z) {
      // z faces are whole padded planes, contiguous per component and already
      // carrying their x / y ghosts (ordered fill): NCCL sends them straight
      // from the field and receives straight into the ghost planes -- no
      // pack / unpack kernels.  Per peer pair the k-th send matches the k-th
      // recv: per component send (hi, lo), recv (lo, hi).
      const Geom& g = ctx->g;
      const size_t pl = (size_t)g.pitch * (size_t)(g.ny + 2 * GUARD);  // one component's x-y plane
      auto plane_ptr = [&](int a, int z) { return f + (size_t)a * g.field + (size_t)(z + GUARD) * (size_t)g.plane; };
      std::vector<XMsg> sends, recvs;
      for (int a = 0; a < ncomp; ++a) {
        if (hi >= 0) sends.push_back({plane_ptr(a, n - 1), pl * sizeof(double), hi});
        if (lo >= 0) sends.push_back({plane_ptr(a, 0), pl * sizeof(double), lo});
      }
      for (int a = 0; a < ncomp; ++a) {
        if (lo >= 0) recvs.push_back({plane_ptr(a, -1), pl * sizeof(double), lo});
        if (hi >= 0) recvs.push_back({plane_ptr(a, n), pl * sizeof(double), hi});
      }
      if (int r = xchg(ctx, sends, recvs, st)) return r;
      if (lo < 0 || hi < 0) {  // physical boundary on one side
        launch_ghost_stage(ctx->g, d, lo < 0 ? ctx->cfg.bc_lo[d] : -1, hi < 0 ? ctx->cfg.bc_hi[d] : -1, f, ncomp, dir,
                           st);
        ctx->nlaunch[2] += 1;
        if (int r = check_launch(ctx, "ghost_stage")) return r;
      }
      continue;
    }
    if (hi >= 0) launch_pack(ctx->g, d, n - 1, ncomp, f, ctx->sendbuf[d][1], st);
    if (lo >= 0) launch_pack(ctx->g, d, 0, ncomp, f, ctx->sendbuf[d][0], st);
    ctx->nlaunch[2] += (hi >= 0) + (lo >= 0);
    if (int r = check_launch(ctx, "pack")) return r;
    if (ctx->collective()) {
      // per peer pair the k-th send matches the k-th recv: send (hi, lo), recv (lo, hi)
      const size_t bytes = cnt * sizeof(double);
      std::vector<XMsg> sends, recvs;
      if (hi >= 0) sends.push_back({ctx->sendbuf[d][1], bytes, hi});
      if (lo >= 0) sends.push_back({ctx->sendbuf[d][0], bytes, lo});
      if (lo >= 0) recvs.push_back({ctx->recvbuf[d][0], bytes, lo});
      if (hi >= 0) recvs.push_back({ctx->recvbuf[d][1], bytes, hi});
      if (int r = xchg(ctx, sends, recvs, st)) return r;
    } else {
      // world == 1, periodic self-exchange through the same pack/unpack path
      CU(cudaMemcpyAsync(ctx->recvbuf[d][0], ctx->sendbuf[d][1], cnt * sizeof(double), cudaMemcpyDeviceToDevice,
                         st));
      CU(cudaMemcpyAsync(ctx->recvbuf[d][1], ctx->sendbuf[d][0], cnt * sizeof(double), cudaMemcpyDeviceToDevice,
                         st));
    }
    if (lo >= 0) launch_unpack(ctx->g, d, -1, ncomp, f, ctx->recvbuf[d][0], st);
    if (hi >= 0) launch_unpack(ctx->g, d, n, ncomp, f, ctx->recvbuf[d][1], st);
    ctx->nlaunch[2] += (hi >= 0) + (lo >= 0);
    if (int r = check_launch(ctx, "unpack")) return r;
    if (lo < 0 || hi < 0) {  // physical boundary on one side of an exchanged dimension
      launch_ghost_stage(ctx->g, d, lo < 0 ? ctx->cfg.bc_lo[d] : -1, hi < 0 ? ctx->cfg.bc_hi[d] : -1, f, ncomp, dir,
                         st);
      ctx->nlaunch[2] += 1;
      if (int r = check_launch(ctx, "ghost_stage")) return r;
    }
  }
  return PF_OK;
}

// kernel choice of a P2 sweep from the tuning (pf_tuning p2_*)
static P2Cfg p2cfg(const pf_tuning& t, bool mu) {
  return mu ? P2Cfg{t.p2_mu, t.p2_mu_ty, t.p2_mu_minb, t.p2_mu_pd, t.p2_mu_hasync}
            : P2Cfg{t.p2_phi, t.p2_phi_ty, t.p2_phi_minb, t.p2_phi_pd, 0};
}

// one P2 sweep with kernel choice c: the run-time specialised kernel
// (PF_VARIANT_JIT, the default: pf_p2_dev.cuh on compile-time parameters)
// or the generic one (PF_VARIANT_TUNED); phi: ps, ms -> pd; mu: ps, pd, ms -> md
static int p2_sweep(pf_ctx* ctx, const P2Cfg& c, bool mu, const double* ps, double* pd, const double* ms,
                    double* md) {
  if (ctx->variant == PF_VARIANT_JIT) {
    const int w = mu ? 1 : 0;
    if (!ctx->jp2[w] || memcmp(&ctx->jp2c[w], &c, sizeof c) != 0) {
      std::string err;
      ctx->jp2[w] = jit_get_p2(ctx, ctx->p2par.data(), ctx->g, c, mu ? P2_MU : P2_PHI, &err);
      if (!ctx->jp2[w]) return fail(ctx, PF_ECUDA, "run-time specialisation of the P2 sweeps failed: %s", err.c_str());
      ctx->jp2c[w] = c;
    }
    CU(mu ? jit_launch_p2(ctx->jp2[w], ctx->dp.Tbase, ps, pd, ms, md, ctx->stream)
          : jit_launch_p2(ctx->jp2[w], ctx->dp.Tbase, ps, ms, nullptr, pd, ctx->stream));
    return PF_OK;
  }
  if (mu)
    p2_launch_mu(ctx->p2par.data(), c, ctx->dp.Tbase, ctx->g, ps, pd, ms, md, ctx->stream);
  else
    p2_launch_phi(ctx->p2par.data(), c, ctx->dp.Tbase, ctx->g, ps, ms, pd, ctx->stream);
  return PF_OK;
}

static int fill_ghosts(pf_ctx* ctx, double* f, int ncomp, bool is_mu, bool x_done = false) {
  return fill_ghost_dims(ctx, f, ncomp, is_mu, 0, 3, ctx->stream, x_done);
}

// make the compute stream wait for an exchange still in flight on comm_s
static int join_comm(pf_ctx* ctx) {
  if (ctx->mux_pending) {
    CU(cudaStreamWaitEvent(ctx->stream, ctx->ev_mux, 0));
    ctx->mux_pending = false;
  }
  return PF_OK;
}


// ---------------------------------------------------------------------------
static cudaEvent_t ev_get(pf_ctx* ctx) {
  if (!ctx->ev_pool.empty()) {
    cudaEvent_t e = ctx->ev_pool.back();
    ctx->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}
static void prof_begin(pf_ctx* ctx, int k, cudaEvent_t* a, cudaStream_t st = nullptr) {
  if (!ctx->prof) return;
  (void)k;
  if (!st) st = ctx->stream;
  if (ctx->cap_sv) {  // capturing a graph: an event-record node of the graph
    cudaEventCreate(a);
    cudaEventRecordWithFlags(*a, st, cudaEventRecordExternal);
    return;
  }
  *a = ev_get(ctx);
  cudaEventRecord(*a, st);
}
static void prof_end(pf_ctx* ctx, int k, cudaEvent_t a, cudaStream_t st = nullptr) {
  if (!ctx->prof) return;
  if (!st) st = ctx->stream;
  if (ctx->cap_sv) {
    cudaEvent_t b = nullptr;
    cudaEventCreate(&b);
    cudaEventRecordWithFlags(b, st, cudaEventRecordExternal);
    ctx->cap_prof.push_back({k, {a, b}});
    return;
  }
  cudaEvent_t b = ev_get(ctx);
  cudaEventRecord(b, st);
  ctx->ev_open.push_back({k, {a, b}});
  if (ctx->ev_open.size() > 4096) {  // drain to bound the pool
    cudaEventSynchronize(b);
    for (auto& o : ctx->ev_open) {
      float ms = 0;
      cudaEventElapsedTime(&ms, o.second.first, o.second.second);
      ctx->prof_ms[o.first] += ms;
      ctx->prof_n[o.first] += 1;
      ctx->ev_pool.push_back(o.second.first);
      ctx->ev_pool.push_back(o.second.second);
    }
    ctx->ev_open.clear();
  }
}

static int window_maybe(pf_ctx* ctx);
static int monitor_check(pf_ctx* ctx, int64_t step_before);
static int front_height_impl(pf_ctx* ctx, int* H);

static int launch_mu(pf_ctx* ctx, const TileSel* ts, dim3 grid, const double* ps, const double* pd,
                     const double* ms, double* md, cudaStream_t st = nullptr) {
  if (st) {  // (the concurrent slab schedule: the specialised sweep on the mu stream)
    CU(jit_launch_mu(ctx->jmu, ctx->dp, ts, grid, ps, pd, ms, md, st, ctx->cap_sv));
    ctx->nlaunch[1] += 1;
    return check_launch(ctx, "mu_sweep");
  }
  if (ctx->variant == PF_VARIANT_NAIVE)
    launch_mu_naive(ctx->dp, ctx->g, ps, pd, ms, md, ctx->stream);
  else if (ctx->variant == PF_VARIANT_SPLIT)
    launch_mu_split(ctx->dp, ctx->g, ps, pd, ms, ctx->stag, md, ctx->stream);
  else if (ctx->variant == PF_VARIANT_JIT)
    CU(jit_launch_mu(ctx->jmu, ctx->dp, ts, grid, ps, pd, ms, md, ctx->stream, ctx->cap_sv));
  else
    launch_mu_tuned(ctx->dp, ctx->g, ts, grid, ps, pd, ms, md, ctx->stream);
  ctx->nlaunch[1] += 1;
  return check_launch(ctx, "mu_sweep");
}

// the z-slab schedule of one step (see step_impl); no exchanged dimension
static int step_slabs(pf_ctx* ctx, const double* ps, double* pd, const double* ms, double* md, bool dry) {
  const Geom& g = ctx->g;
  const int zc = jit_mu_zc_of(ctx->jmu), mty = jit_mu_ty_of(ctx->jmu), mtx = jit_mu_tx_of(ctx->jmu);
  const int H = zc * ctx->tune.slab;
  const int S = (g.nz + H - 1) / H;
  // sched = 2: the mu slabs on their own stream, each after its phi slab and
  // ghosts (an event), so that mu slab s runs concurrently with phi slab s + 1
  // (independent: phi reads phi_src / mu_src, writes other phi_dst planes; mu
  // slab s reads phi_dst planes <= its top + 1, all written by phi slabs <= s)
  // and the two kernels share the SMs; the compute stream joins the mu stream
  // before the mu ghosts
  const bool conc = ctx->tune.sched == 2;
  if (conc) {
    if (!ctx->mu_s) CU(cudaStreamCreateWithFlags(&ctx->mu_s, cudaStreamNonBlocking));
    if (!ctx->ev_slab_done) CU(cudaEventCreateWithFlags(&ctx->ev_slab_done, cudaEventDisableTiming));
    while ((int)ctx->ev_slab.size() < S) {
      cudaEvent_t e = nullptr;
      CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      ctx->ev_slab.push_back(e);
    }
  }
  const dim3 full = tuned_grid_mu(g, mty, zc, mtx);
  BCSpec bxy = ctx->bc_all;  // x / y ghosts of a range of planes: z sides left alone
  bxy.kind_lo[2] = bxy.kind_hi[2] = -1;
  for (int s = 0; s < S; ++s) {
    const int zs = s * H, ze = std::min(g.nz, zs + H);
    const int plo = s == 0 ? 0 : zs + 1, phi_hi = s == S - 1 ? g.nz : ze + 1;
    cudaEvent_t e0 = nullptr;
    prof_begin(ctx, 0, &e0);
    CU(jit_launch_phi(ctx->jphi, ctx->dp, ps, ms, pd, ctx->stream, ctx->cap_sv, plo, phi_hi));
    ctx->nlaunch[0] += 1;
    prof_end(ctx, 0, e0);
    if (int r = check_launch(ctx, "phi_sweep slab")) return r;
    prof_begin(ctx, 2, &e0);
    Geom gs = g;
    gs.nz = phi_hi - plo;
    launch_ghost_fill(gs, bxy, pd + (size_t)plo * (size_t)g.plane, ctx->nph, nullptr, ctx->stream);
    ctx->nlaunch[2] += 1;
    if (s == 0 || s == S - 1) {  // z ghost planes (whole extended planes: after their x / y ghosts)
      launch_ghost_stage(g, 2, s == 0 ? ctx->cfg.bc_lo[2] : -1, s == S - 1 ? ctx->cfg.bc_hi[2] : -1, pd, ctx->nph,
                         nullptr, ctx->stream);
      ctx->nlaunch[2] += 1;
    }
    prof_end(ctx, 2, e0);
    if (int r = check_launch(ctx, "ghost slab")) return r;
    if (s == 0)
      if (int r = join_comm(ctx)) return r;  // the previous step's mu ghosts
    const TileSel ts = {{0, 0, zs / zc}, {0, 0, 0}, {0, 0, 0}, 0};
    cudaStream_t mst = nullptr;
    if (conc) {
      CU(cudaEventRecord(ctx->ev_slab[s], ctx->stream));
      CU(cudaStreamWaitEvent(ctx->mu_s, ctx->ev_slab[s], 0));
      mst = ctx->mu_s;
    }
    prof_begin(ctx, 1, &e0, mst);
    if (int r = launch_mu(ctx, &ts, dim3(full.x, full.y, (unsigned)((ze - zs + zc - 1) / zc)), ps, pd, ms, md, mst))
      return r;
    prof_end(ctx, 1, e0, mst);
  }
  if (conc) {  // join: everything after this waits for the last mu slab
    CU(cudaEventRecord(ctx->ev_slab_done, ctx->mu_s));
    CU(cudaStreamWaitEvent(ctx->stream, ctx->ev_slab_done, 0));
  }
  // line 4: mu ghosts on the side stream (overlapping the next step's first phi slab)
  if (ctx->overlap && ctx->comm_s) {
    CU(cudaEventRecord(ctx->ev_mu, ctx->stream));
    CU(cudaStreamWaitEvent(ctx->comm_s, ctx->ev_mu, 0));
    if (int r = fill_ghost_dims(ctx, md, ctx->nmu, true, 0, 3, ctx->comm_s)) return r;
    CU(cudaEventRecord(ctx->ev_mux, ctx->comm_s));
    ctx->mux_pending = true;
  } else {
    cudaEvent_t e0 = nullptr;
    prof_begin(ctx, 2, &e0);
    const int r = fill_ghosts(ctx, md, ctx->nmu, true);
    prof_end(ctx, 2, e0);
    if (r) return r;
  }
  if (dry) return PF_OK;
  ctx->cur = 1 - ctx->cur;
  ctx->step += 1;
  return PF_OK;
}

// dry = true: every kernel of the step, writing only the scratch level, no
// swap (the state is untouched; pf_autotune times step schedules this way)
static int step_impl(pf_ctx* ctx, bool phi_only, bool dry = false) {
  const Geom& g = ctx->g;
  double* ps = ctx->phi[ctx->cur];
  double* pd = ctx->phi[1 - ctx->cur];
  double* ms = ctx->mu[ctx->cur];
  double* md = ctx->mu[1 - ctx->cur];
  // frozen temperature of this step: T(k) = T0 + G ((k + z0 + z_off) dx - v t_n), t_n = step dt  [A13]
  const double t = (double)ctx->step * ctx->hp.dt;
  ctx->dp.Tbase = ctx->hp.T0 + ctx->hp.G * (((double)g.z0 + (double)ctx->z_off) * ctx->hp.dx - ctx->hp.v * t);
  if (ctx->p2) {
    // P2 (pf_p2.cu): phi-sweep, phi ghosts, mu-sweep, mu ghosts, swap (Algorithm 1)
    if (int r = join_comm(ctx)) return r;
    cudaEvent_t e0 = nullptr;
    prof_begin(ctx, 0, &e0);
    if (int r = p2_sweep(ctx, p2cfg(ctx->tune, false), false, ps, pd, ms, md)) return r;
    ctx->nlaunch[0] += 1;
    prof_end(ctx, 0, e0);
    if (int r = check_launch(ctx, "p2 phi_sweep")) return r;
    prof_begin(ctx, 2, &e0);
    int r = fill_ghosts(ctx, pd, ctx->nph, false);
    prof_end(ctx, 2, e0);
    if (r) return r;
    if (phi_only) {
      CU(cudaMemcpyAsync(md, ms, ctx->lay.mu_bytes - 256, cudaMemcpyDeviceToDevice, ctx->stream));
    } else {
      prof_begin(ctx, 1, &e0);
      if (int r2 = p2_sweep(ctx, p2cfg(ctx->tune, true), true, ps, pd, ms, md)) return r2;
      ctx->nlaunch[1] += 1;
      prof_end(ctx, 1, e0);
      if (int r2 = check_launch(ctx, "p2 mu_sweep")) return r2;
      prof_begin(ctx, 2, &e0);
      r = fill_ghosts(ctx, md, ctx->nmu, true);
      prof_end(ctx, 2, e0);
      if (r) return r;
    }
    if (dry) return PF_OK;
    ctx->cur = 1 - ctx->cur;
    ctx->step += 1;
    return PF_OK;
  }
  ctx->dp.step = (unsigned long long)ctx->step;  // fluctuation counter [B4]
  cudaEvent_t e0 = nullptr;
  if (ctx->variant == PF_VARIANT_JIT && (!ctx->jphi || !ctx->jmu)) {
    std::string err;
    ctx->jphi = jit_get(ctx, ctx->dp, g, ctx->tune, JIT_PHI, &err);
    if (ctx->jphi) ctx->jmu = jit_get(ctx, ctx->dp, g, ctx->tune, JIT_MU, &err);
    if (!ctx->jphi || !ctx->jmu) return fail(ctx, PF_ECUDA, "run-time specialisation failed: %s", err.c_str());
  }
  // overlap: the exchanged dimensions' ghosts travel on the
  // comm stream while the mu-sweep updates the tiles that do not read them
  const bool ov = ctx->overlap && ctx->first_ex < 3 && ctx->variant != PF_VARIANT_NAIVE &&
                  ctx->variant != PF_VARIANT_SPLIT && !phi_only;
  if (ctx->variant == PF_VARIANT_SPLIT && !ctx->stag) {  // the staggered array of the split kernels
    CU(cudaMalloc(&ctx->stag, 12 * (size_t)g.field * sizeof(double) + 256));
  }
  // the specialised phi-sweep writes phi_dst's x ghost columns itself (tuning phi_xghost)
  const bool phi_x_done = g.xwrap && ctx->variant == PF_VARIANT_JIT && ctx->tune.phi_xghost;
  // z-slab schedule (tuning sched = 1, S§7 step 6 (ii)): per slab of mu
  // z-chunks, the phi-sweep of the slab's planes (shifted up by one plane, so
  // that the slab's top neighbour plane is ready), their x/y ghosts, then the
  // mu-sweep of the slab, which re-reads phi_src / phi_dst while the slab is
  // still in L2.  Same kernels and arithmetic per cell as the two sweeps.
  if (ctx->variant == PF_VARIANT_JIT && ctx->tune.sched >= 1 && ctx->first_ex == 3 && !phi_only && !phi_x_done &&
      ctx->cfg.bc_lo[2] != PF_BC_PERIODIC)
    return step_slabs(ctx, ps, pd, ms, md, dry);
  // Algorithm 1, line 1: phi-sweep (reads no mu ghosts: may overlap the previous mu exchange)
  NvtxRange nr_step("pf step: phi-sweep, phi ghosts, mu-sweep, mu ghosts");
  prof_begin(ctx, 0, &e0);
  if (ctx->variant == PF_VARIANT_NAIVE)
    launch_phi_naive(ctx->dp, g, ps, ms, pd, ctx->stream);
  else if (ctx->variant == PF_VARIANT_SPLIT)
    launch_phi_split(ctx->dp, g, ps, ms, ctx->stag, pd, ctx->stream);
  else if (ctx->variant == PF_VARIANT_JIT)
    CU(jit_launch_phi(ctx->jphi, ctx->dp, ps, ms, pd, ctx->stream, ctx->cap_sv));
  else
    launch_phi_tuned(ctx->dp, g, ps, ms, pd, ctx->stream);
  ctx->nlaunch[0] += 1;
  prof_end(ctx, 0, e0);
  if (int r = check_launch(ctx, "phi_sweep")) return r;
  if (!ov) {
    if (int r = join_comm(ctx)) return r;
    // line 2: phi_dst communication and boundary handling
    prof_begin(ctx, 2, &e0);
    int r = fill_ghosts(ctx, pd, ctx->nph, false, phi_x_done);
    prof_end(ctx, 2, e0);
    if (r) return r;
    if (phi_only) {
      CU(cudaMemcpyAsync(md, ms, ctx->lay.mu_bytes - 256, cudaMemcpyDeviceToDevice, ctx->stream));
    } else {
      // line 3: mu-sweep
      prof_begin(ctx, 1, &e0);
      if (int r2 = launch_mu(ctx, nullptr, dim3(), ps, pd, ms, md)) return r2;
      prof_end(ctx, 1, e0);
      // line 4: mu ghosts.  The next phi-sweep reads mu only at its own
      // cells, so the fill runs on the side stream concurrently with it and
      // the next mu-sweep (or any other use) joins first (join_comm).
      if (ctx->overlap && ctx->comm_s) {
        CU(cudaEventRecord(ctx->ev_mu, ctx->stream));
        CU(cudaStreamWaitEvent(ctx->comm_s, ctx->ev_mu, 0));
        if (int r2 = fill_ghost_dims(ctx, md, ctx->nmu, true, 0, 3, ctx->comm_s)) return r2;
        CU(cudaEventRecord(ctx->ev_mux, ctx->comm_s));
        ctx->mux_pending = true;
      } else {
        prof_begin(ctx, 2, &e0);
        r = fill_ghosts(ctx, md, ctx->nmu, true);
        prof_end(ctx, 2, e0);
        if (r) return r;
      }
    }
  } else {
    // line 2: local dimensions before the first exchanged one on the compute
    // stream, the rest (exchanges in x -> y -> z order) on the comm stream
    const int fe = ctx->first_ex;
    if (int r = fill_ghost_dims(ctx, pd, ctx->nph, false, 0, fe, ctx->stream, phi_x_done)) return r;
    CU(cudaEventRecord(ctx->ev_phi, ctx->stream));
    CU(cudaStreamWaitEvent(ctx->comm_s, ctx->ev_phi, 0));
    if (int r = fill_ghost_dims(ctx, pd, ctx->nph, false, fe, 3, ctx->comm_s)) return r;
    CU(cudaEventRecord(ctx->ev_phix, ctx->comm_s));
    // the mu-sweep reads mu ghosts: the previous mu exchange must be done
    if (int r = join_comm(ctx)) return r;
    // line 3: interior tiles (no phi_dst ghost of an exchanged dimension is read)
    const int mty = ctx->variant == PF_VARIANT_JIT ? jit_mu_ty_of(ctx->jmu) : tuned_mu_ty_default();
    const int zc = ctx->variant == PF_VARIANT_JIT ? jit_mu_zc_of(ctx->jmu) : 0;
    const int mtx = ctx->variant == PF_VARIANT_JIT ? jit_mu_tx_of(ctx->jmu) : 32;
    const dim3 full = tuned_grid_mu(g, mty, zc, mtx);
    const int nb[3] = {(int)full.x, (int)full.y, (int)full.z};
    TileSel in = {{0, 0, 0}, {0, 0, 0}, {nb[0], nb[1], nb[2]}, 0};
    bool any_in = true;
    for (int d = fe; d < 3; ++d) {
      in.lo[d] = 1;
      in.hi[d] = nb[d] - 1;
      any_in &= in.hi[d] > in.lo[d];
    }
    prof_begin(ctx, 1, &e0);
    if (any_in) {
      TileSel ti = {{in.lo[0], in.lo[1], in.lo[2]}, {0, 0, 0}, {0, 0, 0}, 0};
      const dim3 gi(in.hi[0] - in.lo[0], in.hi[1] - in.lo[1], in.hi[2] - in.lo[2]);
      if (int r = launch_mu(ctx, &ti, gi, ps, pd, ms, md)) return r;
    }
    // shell tiles once the phi ghosts have arrived
    CU(cudaStreamWaitEvent(ctx->stream, ctx->ev_phix, 0));
    TileSel sh = in;
    sh.skip = any_in ? 1 : 0;
    if (int r = launch_mu(ctx, &sh, full, ps, pd, ms, md)) return r;
    prof_end(ctx, 1, e0);
    // line 4: mu ghosts; the exchange overlaps the next phi-sweep
    if (int r = fill_ghost_dims(ctx, md, ctx->nmu, true, 0, fe, ctx->stream)) return r;
    CU(cudaEventRecord(ctx->ev_mu, ctx->stream));
    CU(cudaStreamWaitEvent(ctx->comm_s, ctx->ev_mu, 0));
    if (int r = fill_ghost_dims(ctx, md, ctx->nmu, true, fe, 3, ctx->comm_s)) return r;
    CU(cudaEventRecord(ctx->ev_mux, ctx->comm_s));
    ctx->mux_pending = true;
  }
  // line 5: swap
  if (dry) return PF_OK;
  ctx->cur = 1 - ctx->cur;
  ctx->step += 1;
  return PF_OK;
}

// k consecutive steps (no window check among them) as one CUDA graph:
// captured on first use for (k, buffer parity), then replayed; the step
// values (T base of each step, step index) go to sv_dev first (one kernel)
static int step_graph(pf_ctx* ctx, int k) {
  if (int r = join_comm(ctx)) return r;
  const Geom& g = ctx->g;
  StepBatch b;
  b.k = k;
  b.step0 = (unsigned long long)ctx->step;
  for (int i = 0; i < k; ++i) {  // the host formula of step_impl, step by step [A13]
    const double t = (double)(ctx->step + i) * ctx->hp.dt;
    b.Tbase[i] = ctx->hp.T0 + ctx->hp.G * (((double)g.z0 + (double)ctx->z_off) * ctx->hp.dx - ctx->hp.v * t);
  }
  launch_set_steps(ctx->sv_dev, b, ctx->stream);
  if (int r = check_launch(ctx, "set_steps")) return r;
  cudaGraphExec_t exec = nullptr;
  pf_ctx::GraphEntry* ge = nullptr;
  for (auto& e : ctx->graphs)
    if (e.k == k && e.cur == ctx->cur) {
      exec = e.exec;
      ge = &e;
    }
  if (ge) graph_prof_collect(ctx, *ge);  // its events are about to be re-recorded
  const int cur0 = ctx->cur;
  const int64_t step0 = ctx->step;
  const int64_t nl[4] = {ctx->nlaunch[0], ctx->nlaunch[1], ctx->nlaunch[2], ctx->nlaunch[3]};
  if (!exec) {
    // capture on the library's own stream (the caller's may be the legacy
    // stream, which cannot be captured); the graph is launched on the caller's.
    // Any failure of the capture falls back to launching the steps directly.
    const cudaStream_t user = ctx->stream;
    cudaGraph_t graph = nullptr;
    ctx->cap_prof.clear();
    cudaError_t e = cudaStreamBeginCapture(ctx->cap_s, cudaStreamCaptureModeThreadLocal);
    int r = e == cudaSuccess ? PF_OK : PF_ECUDA;
    if (r == PF_OK) {
      ctx->stream = ctx->cap_s;
      for (int i = 0; i < k && r == PF_OK; ++i) {
        ctx->cap_sv = ctx->sv_dev + i;
        r = step_impl(ctx, false);
      }
      ctx->cap_sv = nullptr;
      if (r == PF_OK) r = join_comm(ctx);
      ctx->stream = user;
      e = cudaStreamEndCapture(ctx->cap_s, &graph);
      if (r == PF_OK && e == cudaSuccess) e = cudaGraphInstantiate(&exec, graph, 0);
      if (graph) cudaGraphDestroy(graph);
      if (e != cudaSuccess) r = PF_ECUDA;
    }
    // the capture only recorded the steps: rewind the host state
    ctx->cur = cur0;
    ctx->step = step0;
    ctx->mux_pending = false;
    if (r != PF_OK) {
      cudaGetLastError();
      if (exec) cudaGraphExecDestroy(exec);
      for (int i = 0; i < 4; ++i) ctx->nlaunch[i] = nl[i];
      for (auto& pp : ctx->cap_prof) {
        cudaEventDestroy(pp.second.first);
        cudaEventDestroy(pp.second.second);
      }
      ctx->cap_prof.clear();
      ctx->use_graph = false;  // this context steps without graphs from now on
      ctx->err.clear();
      for (int i = 0; i < k; ++i)
        if (int r2 = step_impl(ctx, false)) return r2;
      return PF_OK;
    }
    ctx->graphs.push_back({k, cur0, exec, ctx->cap_prof, false});
    ctx->cap_prof.clear();
    ge = &ctx->graphs.back();
    ctx->mu_launches_per_step = (ctx->nlaunch[1] - nl[1]) / k;
    ctx->ghost_launches_per_step = (ctx->nlaunch[2] - nl[2]) / k;
    for (int i = 0; i < 4; ++i) ctx->nlaunch[i] = nl[i];
  }
  CU(cudaGraphLaunch(exec, ctx->stream));
  ge->pending = !ge->prof.empty();
  for (int i = 0; i < k; ++i) {  // what the k steps did to the host state (step_impl)
    ctx->cur = 1 - ctx->cur;
    ctx->step += 1;
  }
  // launches per category as if the steps had been launched one by one (+ set_steps)
  ctx->nlaunch[0] += k;
  ctx->nlaunch[1] += (int64_t)k * ctx->mu_launches_per_step;
  ctx->nlaunch[2] += (int64_t)k * ctx->ghost_launches_per_step;
  ctx->nlaunch[3] += 1;
  ctx->mux_pending = false;
  return PF_OK;
}

int pf_step(pf_ctx* ctx, int64_t nsteps) {
  if (!ctx) return PF_EINVAL;
  NvtxRange nr("pf_step");
  if (!ctx->have_params || !ctx->have_fields) return fail(ctx, PF_ESTATE, "pf_step before pf_set_params/pf_init_fields");
  if (nsteps < 0) return fail(ctx, PF_EINVAL, "nsteps < 0");
  // graphs pay from ~128^3 cells per block (tools/graph_probe.py: 32^3 slower,
  // 64^3 equal, 256^3 -1.3 % per step); smaller blocks launch directly
  // With pf_profile timing on, steps launch directly unless PF_GRAPH=1 forces
  // graphs (their per-kernel events are then event nodes collected after each
  // replay; measured 0.8 % slower per step at 256^3 than direct profiled steps).
  const bool forced = ctx->graph_min_cells == 0;
  const bool graphs = ctx->use_graph && !ctx->p2 && ctx->variant == PF_VARIANT_JIT && (!ctx->prof || forced) &&
                      (int64_t)ctx->g.nx * ctx->g.ny * ctx->g.nz >= ctx->graph_min_cells;
  // graph runs have one length: the window-check interval (the host decides
  // shifts between runs), else 8 steps; shorter remainders launch directly, so
  // a context captures at most two graphs (one per buffer parity)
  const int nc = ctx->hp.window_check;
  const int64_t K = nc > 0 ? std::min(nc, 64) : 8;
  for (int64_t n = 0; n < nsteps;) {
    int64_t k = 1;
    if (graphs && K >= 2 && nsteps - n >= K && (nc <= 0 || (nc <= 64 && ctx->step % nc == 0))) k = K;
    if (k >= 2) {
      if (ctx->variant == PF_VARIANT_JIT && (!ctx->jphi || !ctx->jmu)) {
        std::string err;
        ctx->jphi = jit_get(ctx, ctx->dp, ctx->g, ctx->tune, JIT_PHI, &err);
        if (ctx->jphi) ctx->jmu = jit_get(ctx, ctx->dp, ctx->g, ctx->tune, JIT_MU, &err);
        if (!ctx->jphi || !ctx->jmu) return fail(ctx, PF_ECUDA, "run-time specialisation failed: %s", err.c_str());
      }
      if (int r = step_graph(ctx, (int)k)) return r;
    } else {
      if (int r = step_impl(ctx, false)) return r;
    }
    n += k;
    if (int r = monitor_check(ctx, ctx->step - k)) return r;
    if (int r = window_maybe(ctx)) return r;
  }
  return join_comm(ctx);
}

int pf_step_phi_only(pf_ctx* ctx) {
  if (!ctx) return PF_EINVAL;
  if (!ctx->have_params || !ctx->have_fields) return fail(ctx, PF_ESTATE, "step before params/fields");
  return step_impl(ctx, true);
}

int pf_halo_exchange(pf_ctx* ctx, unsigned mask) {
  if (!ctx) return PF_EINVAL;
  if (!ctx->have_params) return fail(ctx, PF_ESTATE, "pf_halo_exchange before pf_set_params");
  if (int r = join_comm(ctx)) return r;
  if (mask & PF_PHI)
    if (int r = fill_ghosts(ctx, ctx->phi[ctx->cur], ctx->nph, false)) return r;
  if (mask & PF_MU)
    if (int r = fill_ghosts(ctx, ctx->mu[ctx->cur], ctx->nmu, true)) return r;
  return PF_OK;
}

// ---------------------------------------------------------------------------
int pf_init_fields(pf_ctx* ctx, const double* phi, const double* mu, int where) {
  if (!ctx || !phi || !mu) return PF_EINVAL;
  if (!ctx->have_params) return fail(ctx, PF_ESTATE, "pf_init_fields before pf_set_params");
  const Geom& g = ctx->g;
  const size_t cells = (size_t)g.nx * g.ny * g.nz;
  const cudaMemcpyKind kind = where == PF_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  ctx->cur = 0;
  // stage the packed arrays in the (scratch) second time level, then scatter
  CU(cudaMemcpyAsync(ctx->phi[1], phi, cells * ctx->nph * sizeof(double), kind, ctx->stream));
  CU(cudaMemcpyAsync(ctx->mu[1], mu, cells * ctx->nmu * sizeof(double), kind, ctx->stream));
  launch_copy_interior(g, ctx->nph, ctx->phi[1], ctx->phi[0], 0, ctx->stream);
  launch_copy_interior(g, ctx->nmu, ctx->mu[1], ctx->mu[0], 0, ctx->stream);
  if (int r = check_launch(ctx, "init copy")) return r;
  ctx->step = 0;
  ctx->z_off = 0;
  ctx->have_fields = true;
  // invariants of the input: |sum phi - 1| <= 1e-12, phi >= 0
  double mon[2];
  if (int r = pf_monitor(ctx, mon)) return r;
  if (!(mon[0] <= 1e-12) || !(mon[1] >= 0.0)) {
    ctx->have_fields = false;
    return fail(ctx, PF_EINVAL, "initial fields off the Gibbs simplex or not finite: max|sum phi - 1| = %g, min phi = %g", mon[0], mon[1]);
  }
  if (int r = pf_halo_exchange(ctx, PF_PHI | PF_MU)) return r;
  CU(cudaStreamSynchronize(ctx->stream));
  return PF_OK;
}

int pf_download(pf_ctx* ctx, double* phi, double* mu, int where) {
  if (!ctx || (!phi && !mu)) return PF_EINVAL;
  if (!ctx->have_fields) return fail(ctx, PF_ESTATE, "pf_download before pf_init_fields");
  const Geom& g = ctx->g;
  const size_t cells = (size_t)g.nx * g.ny * g.nz;
  const cudaMemcpyKind kind = where == PF_HOST ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
  // pack into the scratch time level, then copy out
  if (phi) {
    launch_copy_interior(g, ctx->nph, ctx->phi[ctx->cur], ctx->phi[1 - ctx->cur], 1, ctx->stream);
    if (int r = check_launch(ctx, "download copy")) return r;
    CU(cudaMemcpyAsync(phi, ctx->phi[1 - ctx->cur], cells * ctx->nph * sizeof(double), kind, ctx->stream));
  }
  if (mu) {
    launch_copy_interior(g, ctx->nmu, ctx->mu[ctx->cur], ctx->mu[1 - ctx->cur], 1, ctx->stream);
    if (int r = check_launch(ctx, "download copy")) return r;
    CU(cudaMemcpyAsync(mu, ctx->mu[1 - ctx->cur], cells * ctx->nmu * sizeof(double), kind, ctx->stream));
  }
  CU(cudaStreamSynchronize(ctx->stream));
  return PF_OK;
}

int pf_get_state(const pf_ctx* ctx, pf_state* out) {
  if (!ctx || !out) return PF_EINVAL;
  out->step = ctx->step;
  out->z_off = ctx->z_off;
  return PF_OK;
}

int pf_set_state(pf_ctx* ctx, const pf_state* s) {
  if (!ctx || !s || s->step < 0) return PF_EINVAL;
  ctx->step = s->step;
  ctx->z_off = s->z_off;
  return PF_OK;
}

int pf_set_variant(pf_ctx* ctx, int variant) {
  if (!ctx || (variant != PF_VARIANT_TUNED && variant != PF_VARIANT_NAIVE && variant != PF_VARIANT_JIT &&
               variant != PF_VARIANT_SPLIT))
    return PF_EINVAL;
  ctx->variant = variant;
  drop_graphs(ctx);
  return PF_OK;
}

// ---------------------------------------------------------------------------
// reductions (collective over ranks)
// ---------------------------------------------------------------------------
static int allreduce_max_u64(pf_ctx* ctx, unsigned long long* dbuf, int n) {
  return allreduce_max(ctx, dbuf, n);
}

static int front_height_impl(pf_ctx* ctx, int* H) {
  // encode H + 1 >= 0 as u64 so that -1 ("no solid") is the identity of max
  CU(cudaMemsetAsync(ctx->red, 0, 16, ctx->stream));
  launch_front_height(ctx->g, ctx->cfg.liquid, ctx->phi[ctx->cur], (int*)ctx->red, ctx->stream);
  ctx->nlaunch[3] += 1;
  if (int r = check_launch(ctx, "front_height")) return r;
  if (int r = allreduce_max_u64(ctx, ctx->red, 1)) return r;
  CU(cudaMemcpyAsync(ctx->pinned, ctx->red, 8, cudaMemcpyDeviceToHost, ctx->stream));
  CU(cudaStreamSynchronize(ctx->stream));
  *H = (int)(ctx->pinned[0] & 0xffffffffull) - 1;
  return PF_OK;
}

int pf_front_height(pf_ctx* ctx, int* H) {
  if (!ctx || !H) return PF_EINVAL;
  if (!ctx->have_fields) return fail(ctx, PF_ESTATE, "no fields");
  return front_height_impl(ctx, H);
}

int pf_set_monitors(pf_ctx* ctx, int every, double tol) {
  if (!ctx) return PF_EINVAL;
  if (every < 0 || !(tol >= 0.0)) return fail(ctx, PF_EINVAL, "pf_set_monitors: every >= 0, tol >= 0");
  ctx->mon_every = every;
  ctx->mon_tol = tol;
  return PF_OK;
}

// inside pf_step: the monitors after a run of steps that reached a multiple of mon_every
static int monitor_check(pf_ctx* ctx, int64_t step_before) {
  if (ctx->mon_every <= 0 || ctx->step / ctx->mon_every == step_before / ctx->mon_every) return PF_OK;
  double m[2];
  if (int r = pf_monitor(ctx, m)) return r;
  if (!(m[0] <= ctx->mon_tol) || !(m[1] >= -ctx->mon_tol))
    return fail(ctx, PF_ENUMERIC, "monitor tripped after step %lld: max|sum phi - 1| = %g, min phi = %g (tol %g)",
                (long long)ctx->step, m[0], m[1], ctx->mon_tol);
  return PF_OK;
}

int pf_monitor(pf_ctx* ctx, double out[2]) {
  if (!ctx || !out) return PF_EINVAL;
  if (!ctx->have_fields) return fail(ctx, PF_ESTATE, "no fields");
  CU(cudaMemsetAsync(ctx->red, 0, 16, ctx->stream));
  launch_monitor(ctx->g, ctx->nph, ctx->nmu, ctx->phi[ctx->cur], ctx->mu[ctx->cur], ctx->red, ctx->stream);
  if (int r = check_launch(ctx, "monitor")) return r;
  if (int r = allreduce_max_u64(ctx, ctx->red, 2)) return r;
  CU(cudaMemcpyAsync(ctx->pinned, ctx->red, 16, cudaMemcpyDeviceToHost, ctx->stream));
  CU(cudaStreamSynchronize(ctx->stream));
  auto dec = [](unsigned long long b) {
    b = (b & 0x8000000000000000ull) ? (b & 0x7fffffffffffffffull) : ~b;
    double v;
    memcpy(&v, &b, 8);
    return v;
  };
  out[0] = dec(ctx->pinned[0]);
  out[1] = -dec(ctx->pinned[1]);
  return PF_OK;
}

// ---------------------------------------------------------------------------
// moving window (S6) [A16]
// ---------------------------------------------------------------------------
int pf_shift_window(pf_ctx* ctx, int k) {
  if (!ctx) return PF_EINVAL;
  if (!ctx->have_fields) return fail(ctx, PF_ESTATE, "no fields");
  const int pz = ctx->cfg.procs[2] < 1 ? 1 : ctx->cfg.procs[2];
  if (pz != 1) return fail(ctx, PF_EINVAL, "the moving window needs the growth axis unsplit (procs[2] == 1)");
  if (k < 0 || k > ctx->g.nz) return fail(ctx, PF_EINVAL, "shift %d out of range", k);
  if (k == 0) return PF_OK;
  if (int r = join_comm(ctx)) return r;
  cudaEvent_t e0 = nullptr;
  prof_begin(ctx, 3, &e0);
  launch_shift(ctx->g, k, ctx->cfg.liquid, ctx->nph, ctx->nmu, ctx->hp.mu_inf, ctx->phi[ctx->cur], ctx->mu[ctx->cur],
               ctx->phi[1 - ctx->cur], ctx->mu[1 - ctx->cur], ctx->stream);
  ctx->nlaunch[3] += 1;
  prof_end(ctx, 3, e0);
  if (int r = check_launch(ctx, "shift")) return r;
  ctx->cur = 1 - ctx->cur;
  ctx->z_off += k;
  return pf_halo_exchange(ctx, PF_PHI | PF_MU);
}

static int window_maybe(pf_ctx* ctx) {
  NvtxRange nr("pf window check");
  const int nc = ctx->hp.window_check;
  if (nc <= 0 || ctx->step % nc != 0) return PF_OK;
  int H = -1;
  if (int r = front_height_impl(ctx, &H)) return r;
  const int thr = (int)floor(ctx->hp.window_frac * (double)ctx->cfg.global[2]);
  if (H > thr) return pf_shift_window(ctx, H - thr);
  return PF_OK;
}

// ---------------------------------------------------------------------------
// tuning and auto-tuning of the specialised sweeps (S§8(f) NEXT-2;
// P:L797-806 mapping auto-tuning, P:L808-865 per-kernel tuning)
// ---------------------------------------------------------------------------
int pf_tuning_default(pf_tuning* out) {
  if (!out) return PF_EINVAL;
  tuning_default(out);
  return PF_OK;
}

int pf_set_tuning(pf_ctx* ctx, const pf_tuning* t) {
  if (!ctx || !t) return PF_EINVAL;
  if (const char* m = tuning_check(*t)) return fail(ctx, PF_EINVAL, "pf_set_tuning: %s", m);
  ctx->tune = *t;
  ctx->jphi = ctx->jmu = ctx->jp2[0] = ctx->jp2[1] = nullptr;
  drop_graphs(ctx);
  return PF_OK;
}

int pf_get_tuning(const pf_ctx* ctx, pf_tuning* out) {
  if (!ctx || !out) return PF_EINVAL;
  *out = ctx->tune;
  return PF_OK;
}

namespace {
struct TuneKnob {
  const char* name;
  int pf_tuning::*f;
  int which;
  std::vector<int> dom;
};
const std::vector<TuneKnob>& tune_knobs() {
  static const std::vector<TuneKnob> k = {
      {"phi_ty", &pf_tuning::phi_ty, JIT_PHI, {4, 8, 16}},
      {"phi_minb", &pf_tuning::phi_minb, JIT_PHI, {3, 4, 5, 6}},
      {"phi_zc", &pf_tuning::phi_zc, JIT_PHI, {8, 12, 16, 24, 32}},
      {"phi_faces6", &pf_tuning::phi_faces6, JIT_PHI, {0, 1}},
      {"phi_unroll", &pf_tuning::phi_unroll, JIT_PHI, {1, 2, 3}},
      {"phi_prefetch", &pf_tuning::phi_prefetch, JIT_PHI, {0, 1, 2}},
      {"phi_pfd", &pf_tuning::phi_pfd, JIT_PHI, {1, 2, 3}},
      {"phi_xsh", &pf_tuning::phi_xsh, JIT_PHI, {0, 1}},
      {"phi_zrec", &pf_tuning::phi_zrec, JIT_PHI, {0, 1}},
      {"phi_xghost", &pf_tuning::phi_xghost, JIT_PHI, {0, 1}},
      {"mu_ty", &pf_tuning::mu_ty, JIT_MU, {3, 4, 5, 6, 8}},
      {"mu_tx", &pf_tuning::mu_tx, JIT_MU, {16, 32}},
      {"mu_minb", &pf_tuning::mu_minb, JIT_MU, {2, 3, 4}},
      {"mu_zc", &pf_tuning::mu_zc, JIT_MU, {8, 12, 16, 22, 24, 32}},
      {"mu_prefetch", &pf_tuning::mu_prefetch, JIT_MU, {0, 1, 2}},
      {"mu_pfd", &pf_tuning::mu_pfd, JIT_MU, {2, 3, 4, 6}},
      {"mu_rpf", &pf_tuning::mu_rpf, JIT_MU, {0, 1}},
      {"mu_halo_l1", &pf_tuning::mu_halo_l1, JIT_MU, {0, 1}},
      {"mu_fxreg", &pf_tuning::mu_fxreg, JIT_MU, {0, 1}},
      {"mu_qreg", &pf_tuning::mu_qreg, JIT_MU, {0, 1}},
      {"mu_ldhint", &pf_tuning::mu_ldhint, JIT_MU, {0, 1, 2, 3}},
      {"mu_hpipe", &pf_tuning::mu_hpipe, JIT_MU, {0, 1}},
      {"mu_cly", &pf_tuning::mu_cly, JIT_MU, {1, 2, 4}},
      {"mu_rot", &pf_tuning::mu_rot, JIT_MU, {0, 1}},
      {"mu_rpt", &pf_tuning::mu_rpt, JIT_MU, {1, 2}},
      {"phi_rpt", &pf_tuning::phi_rpt, JIT_PHI, {1, 2}},
      {"mu_pers", &pf_tuning::mu_pers, JIT_MU, {0, 1}},
      {"phi_pers", &pf_tuning::phi_pers, JIT_PHI, {0, 1}},
      {"mu_tmem", &pf_tuning::mu_tmem, JIT_MU, {0, 1}},
      {"mu_hcar", &pf_tuning::mu_hcar, JIT_MU, {0, 1}},
      {"mu_xshfl", &pf_tuning::mu_xshfl, JIT_MU, {0, 1}},
      {"mu_hasync", &pf_tuning::mu_hasync, JIT_MU, {0, 1, 2}},
      // P2 (pf_p2.cu): tuned by the P2 branch of pf_autotune
      {"p2_phi", &pf_tuning::p2_phi, P2_PHI, {0, 1, 2}},
      {"p2_mu", &pf_tuning::p2_mu, P2_MU, {0, 1, 2}},
      {"p2_phi_ty", &pf_tuning::p2_phi_ty, P2_PHI, {4, 8}},
      {"p2_phi_minb", &pf_tuning::p2_phi_minb, P2_PHI, {1, 2, 3, 4}},
      {"p2_mu_ty", &pf_tuning::p2_mu_ty, P2_MU, {4, 8}},
      {"p2_mu_minb", &pf_tuning::p2_mu_minb, P2_MU, {1, 2, 3, 4}},
      {"p2_phi_pd", &pf_tuning::p2_phi_pd, P2_PHI, {0, 1, 2, 3, 4}},
      {"p2_mu_pd", &pf_tuning::p2_mu_pd, P2_MU, {0, 1, 2, 3, 4}},
      {"p2_mu_hasync", &pf_tuning::p2_mu_hasync, P2_MU, {0, 1}},
      // not searched (data-dependent time; reported separately by bench.py)
      {"mu_atskip", &pf_tuning::mu_atskip, JIT_MU, {0}},
  };
  return k;
}

std::string tuning_json(const pf_tuning& t) {
  std::string o = "{";
  bool first = true;
  for (const auto& k : tune_knobs()) {
    char b[64];
    snprintf(b, sizeof b, "%s\"%s\": %d", first ? "" : ", ", k.name, t.*(k.f));
    o += b;
    first = false;
  }
  // the step schedule (timed as whole dry steps, not a per-kernel knob)
  char b[64];
  snprintf(b, sizeof b, ", \"sched\": %d, \"slab\": %d", t.sched, t.slab);
  return o + b + "}";
}
}  // namespace

// median launch time (ms) of one specialised sweep on this context's fields;
// reads only the current level, writes only the scratch level
static int time_sweep(pf_ctx* ctx, JitKernel* k, int which, int reps, double* out) {
  const double* ps = ctx->phi[ctx->cur];
  double* pd = ctx->phi[1 - ctx->cur];
  const double* ms = ctx->mu[ctx->cur];
  double* md = ctx->mu[1 - ctx->cur];
  auto launch = [&]() {
    return which == JIT_PHI ? jit_launch_phi(k, ctx->dp, ps, ms, pd, ctx->stream)
                            : jit_launch_mu(k, ctx->dp, nullptr, dim3(), ps, pd, ms, md, ctx->stream);
  };
  for (int i = 0; i < 2; ++i) CU(launch());
  std::vector<cudaEvent_t> ev(reps + 1);
  for (auto& e : ev) CU(cudaEventCreate(&e));
  CU(cudaEventRecord(ev[0], ctx->stream));
  for (int i = 0; i < reps; ++i) {
    CU(launch());
    CU(cudaEventRecord(ev[i + 1], ctx->stream));
  }
  CU(cudaEventSynchronize(ev[reps]));
  std::vector<double> t(reps);
  for (int i = 0; i < reps; ++i) {
    float v = 0;
    cudaEventElapsedTime(&v, ev[i], ev[i + 1]);
    t[i] = v;
  }
  for (auto e : ev) cudaEventDestroy(e);
  std::sort(t.begin(), t.end());
  *out = t[reps / 2];
  return PF_OK;
}

// P2 (pf_p2.cu): every kernel choice of each sweep (p2_* knobs: kernel,
// side-staged tile height x CTAs per SM, prefetch distance), each timed as
// the median of `reps` launches on this context's fields (reads the current
// level, writes the scratch level: the state is untouched); the times are
// max-reduced over ranks so that every rank keeps the same choice; a
// candidate replaces the current choice only if >= 1 % faster
static int time_p2(pf_ctx* ctx, const pf_tuning& t, bool mu, int reps, double* out) {
  const double* ps = ctx->phi[ctx->cur];
  double* pd = ctx->phi[1 - ctx->cur];
  const double* ms = ctx->mu[ctx->cur];
  double* md = ctx->mu[1 - ctx->cur];
  const P2Cfg c = p2cfg(t, mu);
  auto launch = [&]() -> cudaError_t {
    if (p2_sweep(ctx, c, mu, ps, pd, ms, md) != PF_OK) return cudaErrorLaunchFailure;
    return cudaGetLastError();
  };
  if (int r = p2_sweep(ctx, c, mu, ps, pd, ms, md)) return r;  // (compiles / loads the specialised kernel)
  for (int i = 0; i < 2; ++i) CU(launch());
  std::vector<cudaEvent_t> ev(reps + 1);
  for (auto& e : ev) CU(cudaEventCreate(&e));
  CU(cudaEventRecord(ev[0], ctx->stream));
  for (int i = 0; i < reps; ++i) {
    CU(launch());
    CU(cudaEventRecord(ev[i + 1], ctx->stream));
  }
  CU(cudaEventSynchronize(ev[reps]));
  std::vector<double> tm(reps);
  for (int i = 0; i < reps; ++i) {
    float v = 0;
    cudaEventElapsedTime(&v, ev[i], ev[i + 1]);
    tm[i] = v;
  }
  for (auto e : ev) cudaEventDestroy(e);
  std::sort(tm.begin(), tm.end());
  *out = tm[reps / 2];
  return PF_OK;
}

static int autotune_p2(pf_ctx* ctx, unsigned mask, int reps, char* log, int logn) {
  if (!(mask & (PF_PHI | PF_MU)) || reps < 1 || reps > 1000)
    return fail(ctx, PF_EINVAL, "pf_autotune: mask PF_PHI|PF_MU, 1 <= reps <= 1000");
  if (int r = join_comm(ctx)) return r;
  CU(cudaStreamSynchronize(ctx->stream));
  const pf_tuning start = ctx->tune;
  pf_tuning best = start;
  std::string cl, kj;
  for (bool mu : {false, true}) {
    if (!(mask & (mu ? PF_MU : PF_PHI))) continue;
    if (mu) {  // the mu-sweep reads phi_dst: one phi-sweep of the chosen phi kernel and its ghosts first
      if (int r = p2_sweep(ctx, p2cfg(best, false), false, ctx->phi[ctx->cur], ctx->phi[1 - ctx->cur],
                           ctx->mu[ctx->cur], ctx->mu[1 - ctx->cur]))
        return r;
      CU(cudaGetLastError());
      if (int r = fill_ghosts(ctx, ctx->phi[1 - ctx->cur], ctx->nph, false)) return r;
    }
    std::vector<pf_tuning> cands{best};
    for (int k : {0, 1, 2})
      for (int tm : {0, 1, 2, 3, 4, 5})
        for (int pdist : {0, 1, 2, 3, 4})
        for (int ha : {0, 1}) {
          if (k != 0 && (tm || pdist || ha)) continue;  // tile / prefetch / staging only matter for the side-staged kernels
          if (ha && (!mu || ctx->variant != PF_VARIANT_JIT || tm < 2)) continue;  // (staging: the specialised mu kernel, 32 x 4 tiles)
          pf_tuning c = best;
          if (mu) c.p2_mu_hasync = ha;
          const int ty = tm < 2 ? 8 : 4, mb = tm == 0 ? 2 : tm == 1 ? 1 : tm + 1;  // 8x2 8x1 4x3 4x4 4x5 4x6
          (mu ? c.p2_mu : c.p2_phi) = k;
          if (k == 0) {
            (mu ? c.p2_mu_ty : c.p2_phi_ty) = ty;
            (mu ? c.p2_mu_minb : c.p2_phi_minb) = mb;
            (mu ? c.p2_mu_pd : c.p2_phi_pd) = pdist;
          }
          if (!tuning_check(c) && memcmp(&c, &best, sizeof c)) cands.push_back(c);
        }
    if (ctx->variant == PF_VARIANT_JIT) {  // every candidate's specialised kernel, on host threads
      std::vector<std::string> srcs;
      for (const auto& c : cands) srcs.push_back(p2_specialised_source(ctx->p2par.data(), ctx->g, p2cfg(c, mu), mu ? P2_MU : P2_PHI));
      jit_precompile_sources(srcs, (int)std::max(1u, std::thread::hardware_concurrency()));
    }
    std::vector<double> tms(cands.size(), INFINITY);
    for (size_t i = 0; i < cands.size(); ++i)
      if (int r = time_p2(ctx, cands[i], mu, reps, &tms[i])) return r;
    if (ctx->collective()) {
      double* d = (double*)ctx->red;
      const int n = (int)cands.size();
      CU(cudaMemcpyAsync(d, tms.data(), n * sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
      if (int r = allreduce_max(ctx, d, n)) return r;
      CU(cudaMemcpyAsync(tms.data(), d, n * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
      CU(cudaStreamSynchronize(ctx->stream));
    }
    size_t bi = 0;
    for (size_t i = 1; i < cands.size(); ++i)
      if (tms[i] < tms[0] * 0.99 && tms[i] < tms[bi]) bi = i;
    const char* kname = mu ? "mu" : "phi";
    for (size_t i = 1; i < cands.size(); ++i) {
      const pf_tuning& c = cands[i];
      char b[320];
      snprintf(b, sizeof b,
               "%s{\"kernel\": \"p2_%s\", \"pass\": 0, \"knob\": \"kern/ty/minb/pd\", \"value\": %d, \"ms\": %.6f, \"error\": \"\"}",
               cl.empty() ? "" : ",\n  ", kname,
               1000 * (mu ? c.p2_mu : c.p2_phi) + 100 * (mu ? c.p2_mu_ty : c.p2_phi_ty) +
                   10 * (mu ? c.p2_mu_minb : c.p2_phi_minb) + (mu ? c.p2_mu_pd : c.p2_phi_pd),
               tms[i]);
      cl += b;
    }
    best = cands[bi];
    char b[256];
    snprintf(b, sizeof b, "%s\"%s\": {\"start_ms\": %.6f, \"best_ms\": %.6f, \"candidates\": %d}", kj.empty() ? "" : ", ",
             kname, tms[0], tms[bi], (int)cands.size() - 1);
    kj += b;
  }
  ctx->tune = best;
  CU(cudaStreamSynchronize(ctx->stream));
  if (log && logn > 0) {
    std::string j = "{\"start\": " + tuning_json(start) + ",\n \"best\": " + tuning_json(best) + ",\n " + kj +
                    ",\n \"reps\": " + std::to_string(reps) + ",\n \"tried\": [\n  " + cl + "]}";
    snprintf(log, (size_t)logn, "%s", j.c_str());
  }
  return PF_OK;
}

// median time of one dry step (all kernels of a step on the scratch level)
static int time_steps(pf_ctx* ctx, int reps, double* out) {
  for (int i = 0; i < 2; ++i)
    if (int r = step_impl(ctx, false, true)) return r;
  std::vector<cudaEvent_t> ev(reps + 1);
  for (auto& e : ev) CU(cudaEventCreate(&e));
  CU(cudaEventRecord(ev[0], ctx->stream));
  for (int i = 0; i < reps; ++i) {
    if (int r = step_impl(ctx, false, true)) return r;
    if (int r = join_comm(ctx)) return r;
    CU(cudaEventRecord(ev[i + 1], ctx->stream));
  }
  CU(cudaEventSynchronize(ev[reps]));
  std::vector<double> t(reps);
  for (int i = 0; i < reps; ++i) {
    float v = 0;
    cudaEventElapsedTime(&v, ev[i], ev[i + 1]);
    t[i] = v;
  }
  for (auto e : ev) cudaEventDestroy(e);
  std::sort(t.begin(), t.end());
  *out = t[reps / 2];
  return PF_OK;
}

// times of candidate kernels (inf where the build failed), max over ranks
static int time_candidates(pf_ctx* ctx, const std::vector<pf_tuning>& cands, int which, int reps,
                           std::vector<double>* ms, std::vector<std::string>* why) {
  const int nthr = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  jit_precompile(ctx->dp, ctx->g, cands, which, nthr);
  ms->assign(cands.size(), INFINITY);
  why->assign(cands.size(), "");
  for (size_t i = 0; i < cands.size(); ++i) {
    std::string err;
    JitKernel* k = jit_get(ctx, ctx->dp, ctx->g, cands[i], which, &err);
    if (!k) {
      (*why)[i] = err.substr(0, 200);
      continue;
    }
    double v = INFINITY;
    if (int r = time_sweep(ctx, k, which, reps, &v)) {
      cudaGetLastError();  // e.g. a launch the tile shape cannot fit: not sticky
      (*why)[i] = "launch failed";
      (void)r;
      continue;
    }
    (*ms)[i] = v;
  }
  if (ctx->collective()) {  // every rank takes the same decision: max over ranks
    double* d = (double*)ctx->red;
    for (size_t o = 0; o < cands.size(); o += 32) {
      const size_t n = std::min<size_t>(32, cands.size() - o);
      CU(cudaMemcpyAsync(d, ms->data() + o, n * sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
      if (int r = allreduce_max(ctx, d, (int)n)) return r;
      CU(cudaMemcpyAsync(ms->data() + o, d, n * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
      CU(cudaStreamSynchronize(ctx->stream));
    }
  }
  return PF_OK;
}

int pf_autotune(pf_ctx* ctx, unsigned mask, int passes, int reps, char* log, int logn) {
  if (!ctx) return PF_EINVAL;
  if (!ctx->have_params || !ctx->have_fields) return fail(ctx, PF_ESTATE, "pf_autotune before pf_set_params/pf_init_fields");
  if (ctx->p2) return autotune_p2(ctx, mask, reps, log, logn);
  if (ctx->variant != PF_VARIANT_JIT) return fail(ctx, PF_ESTATE, "pf_autotune tunes the JIT variant (or a P2 context)");
  if (!(mask & (PF_PHI | PF_MU)) || passes < 1 || reps < 1 || reps > 1000)
    return fail(ctx, PF_EINVAL, "pf_autotune: mask PF_PHI|PF_MU, passes >= 1, 1 <= reps <= 1000");
  if (const char* m = tuning_check(ctx->tune)) return fail(ctx, PF_EINVAL, "current tuning invalid: %s", m);
  if (int r = join_comm(ctx)) return r;
  CU(cudaStreamSynchronize(ctx->stream));
  const pf_tuning start = ctx->tune;
  pf_tuning best = start;
  std::string cl;  // candidate records
  std::string kj;  // per-kernel summary
  for (int which : {JIT_PHI, JIT_MU}) {
    if (!(mask & (which == JIT_PHI ? PF_PHI : PF_MU))) continue;
    const char* kname = which == JIT_PHI ? "phi" : "mu";
    if (which == JIT_MU) {  // the mu-sweep reads phi_dst: one phi-sweep of the best phi kernel first
      std::string err;
      JitKernel* kp = jit_get(ctx, ctx->dp, ctx->g, best, JIT_PHI, &err);
      if (!kp) return fail(ctx, PF_ECUDA, "autotune: %s", err.c_str());
      CU(jit_launch_phi(kp, ctx->dp, ctx->phi[ctx->cur], ctx->mu[ctx->cur], ctx->phi[1 - ctx->cur], ctx->stream));
      if (int r = fill_ghosts(ctx, ctx->phi[1 - ctx->cur], ctx->nph, false)) return r;
    }
    std::vector<double> t0;
    std::vector<std::string> w0;
    if (int r = time_candidates(ctx, {best}, which, reps, &t0, &w0)) return r;
    if (!std::isfinite(t0[0])) return fail(ctx, PF_ECUDA, "autotune: the current %s kernel failed: %s", kname, w0[0].c_str());
    const double start_ms = t0[0];
    double best_ms = start_ms;
    int ncand = 0;
    for (int pass = 0; pass < passes; ++pass) {
      bool improved = false;
      for (const auto& kn : tune_knobs()) {
        if (kn.which != which) continue;
        std::vector<pf_tuning> cands;
        std::vector<int> vals;
        for (int v : kn.dom) {
          if (v == best.*(kn.f)) continue;
          pf_tuning c = best;
          c.*(kn.f) = v;
          // a new tile shape comes with its natural occupancy
          if (kn.f == &pf_tuning::phi_rpt) c.phi_ty = v == 2 ? 8 : 4;
          if (kn.f == &pf_tuning::phi_ty || kn.f == &pf_tuning::phi_rpt) c.phi_minb = phi_minb_for(c.phi_ty, c.phi_rpt);
          // (two rows per thread come with their natural 32 x 8 tile, one row with 32 x 4)
          if (kn.f == &pf_tuning::mu_rpt) c.mu_ty = v == 2 ? 8 : 4;
          if (kn.f == &pf_tuning::mu_ty || kn.f == &pf_tuning::mu_tx || kn.f == &pf_tuning::mu_rpt)
            c.mu_minb = mu_minb_for(c.mu_ty, c.mu_tx, c.mu_rpt);
          if (tuning_check(c)) continue;
          cands.push_back(c);
          vals.push_back(v);
        }
        if (cands.empty()) continue;
        std::vector<double> tm;
        std::vector<std::string> why;
        if (int r = time_candidates(ctx, cands, which, reps, &tm, &why)) return r;
        int bi = -1;
        for (size_t i = 0; i < cands.size(); ++i) {
          char b[512];
          snprintf(b, sizeof b, "%s{\"kernel\": \"%s\", \"pass\": %d, \"knob\": \"%s\", \"value\": %d, \"ms\": %s, \"error\": \"%s\"}",
                   cl.empty() ? "" : ",\n  ", kname, pass, kn.name, vals[i],
                   std::isfinite(tm[i]) ? std::to_string(tm[i]).c_str() : "null", why[i].c_str());
          cl += b;
          ++ncand;
          if (tm[i] < best_ms * 0.99 && (bi < 0 || tm[i] < tm[bi])) bi = (int)i;
        }
        if (bi >= 0) {
          best = cands[bi];
          best_ms = tm[bi];
          improved = true;
        }
      }
      if (!improved) break;
    }
    char b[256];
    snprintf(b, sizeof b, "%s\"%s\": {\"start_ms\": %.6f, \"best_ms\": %.6f, \"candidates\": %d}", kj.empty() ? "" : ", ",
             kname, start_ms, best_ms, ncand);
    kj += b;
  }
  ctx->tune = best;
  ctx->jphi = ctx->jmu = ctx->jp2[0] = ctx->jp2[1] = nullptr;
  drop_graphs(ctx);
  {
    std::string err;
    ctx->jphi = jit_get(ctx, ctx->dp, ctx->g, best, JIT_PHI, &err);
    if (ctx->jphi) ctx->jmu = jit_get(ctx, ctx->dp, ctx->g, best, JIT_MU, &err);
    if (!ctx->jphi || !ctx->jmu) return fail(ctx, PF_ECUDA, "autotune: %s", err.c_str());
  }
  // step schedule (S§8(f) NEXT-2 "full vs split vs fused schedules"): two
  // sweeps vs the z-slab pipeline, timed as whole dry steps (every kernel of
  // a step, scratch level only, no swap)
  const bool slab_ok = (mask & PF_PHI) && (mask & PF_MU) && ctx->first_ex == 3 &&
                       ctx->cfg.bc_lo[2] != PF_BC_PERIODIC && !(ctx->g.xwrap && ctx->tune.phi_xghost);
  if (slab_ok) {
    std::vector<pf_tuning> cands;
    for (int sc : {0, 1, 2})
      for (int sl : {1, 2, 4}) {
        if (sc == 0 && sl != 1) continue;
        pf_tuning c = best;
        c.sched = sc;
        c.slab = sc ? sl : best.slab;
        if (!tuning_check(c)) cands.push_back(c);
      }
    std::vector<double> tm(cands.size(), INFINITY);
    for (size_t i = 0; i < cands.size(); ++i) {
      ctx->tune = cands[i];
      double v = INFINITY;
      if (int r = time_steps(ctx, reps, &v)) return r;
      tm[i] = v;
    }
    if (ctx->collective()) {
      double* d = (double*)ctx->red;
      const int n = (int)cands.size();
      CU(cudaMemcpyAsync(d, tm.data(), n * sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
      if (int r = allreduce_max(ctx, d, n)) return r;
      CU(cudaMemcpyAsync(tm.data(), d, n * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
      CU(cudaStreamSynchronize(ctx->stream));
    }
    size_t bi = 0;
    for (size_t i = 0; i < cands.size(); ++i) {
      if (tm[i] < tm[bi] * 0.99) bi = i;
      char b[256];
      snprintf(b, sizeof b, "%s{\"kernel\": \"step\", \"pass\": 0, \"knob\": \"sched/slab\", \"value\": %d, \"ms\": %s, \"error\": \"\"}",
               cl.empty() ? "" : ",\n  ", cands[i].sched ? cands[i].slab : 0,
               std::isfinite(tm[i]) ? std::to_string(tm[i]).c_str() : "null");
      cl += b;
    }
    best = cands[bi];
    ctx->tune = best;
    char b[256];
    snprintf(b, sizeof b, ", \"step\": {\"two_sweeps_ms\": %.6f, \"best_ms\": %.6f, \"sched\": %d, \"slab\": %d}", tm[0],
             tm[bi], best.sched, best.slab);
    kj += b;
    if (mask & PF_AUTOTUNE_VARIANTS) {
      // kernel variants of the paper: full (every face flux
      // evaluated by both cells) and split (staggered fluxes through a global
      // array) against the fused on-chip JIT sweeps, as whole dry steps
      double tj = tm[bi], tv[2] = {INFINITY, INFINITY};
      const int vs[2] = {PF_VARIANT_NAIVE, PF_VARIANT_SPLIT};
      for (int i = 0; i < 2; ++i) {
        ctx->variant = vs[i];
        if (int r = time_steps(ctx, reps, &tv[i])) {
          ctx->variant = PF_VARIANT_JIT;
          return r;
        }
      }
      if (ctx->collective()) {
        double* d = (double*)ctx->red;
        CU(cudaMemcpyAsync(d, tv, 2 * sizeof(double), cudaMemcpyHostToDevice, ctx->stream));
        if (int r = allreduce_max(ctx, d, 2)) return r;
        CU(cudaMemcpyAsync(tv, d, 2 * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
        CU(cudaStreamSynchronize(ctx->stream));
      }
      ctx->variant = PF_VARIANT_JIT;
      if (tv[0] < tj * 0.99 || tv[1] < tj * 0.99) ctx->variant = tv[0] < tv[1] ? vs[0] : vs[1];
      snprintf(b, sizeof b,
               ", \"variants\": {\"fused_jit_ms\": %.6f, \"full_ms\": %.6f, \"split_ms\": %.6f, \"chosen\": %d}", tj,
               tv[0], tv[1], ctx->variant);
      kj += b;
    }
  }
  // the scratch level's ghosts were overwritten: nothing reads them before the next sweep writes it
  CU(cudaStreamSynchronize(ctx->stream));
  if (log && logn > 0) {
    std::string j = "{\"start\": " + tuning_json(start) + ",\n \"best\": " + tuning_json(best) + ",\n " + kj +
                    ",\n \"reps\": " + std::to_string(reps) + ",\n \"tried\": [\n  " + cl + "]}";
    snprintf(log, (size_t)logn, "%s", j.c_str());
  }
  return PF_OK;
}

// ---------------------------------------------------------------------------
int pf_profile(pf_ctx* ctx, int enable) {
  if (!ctx) return PF_EINVAL;
  CU(cudaStreamSynchronize(ctx->stream));
  if ((enable != 0) != ctx->prof) {
    drop_graphs(ctx);  // graphs are re-captured with (or without) their timing events
  } else {
    for (auto& e : ctx->graphs) e.pending = false;  // discard the replays before the reset
  }
  for (auto& o : ctx->ev_open) {
    ctx->ev_pool.push_back(o.second.first);
    ctx->ev_pool.push_back(o.second.second);
  }
  ctx->ev_open.clear();
  for (int i = 0; i < 4; ++i) {
    ctx->prof_ms[i] = 0;
    ctx->prof_n[i] = 0;
    ctx->nlaunch[i] = 0;
  }
  ctx->prof = enable != 0;
  return PF_OK;
}

int pf_profile_read(pf_ctx* ctx, double ms[4], int64_t launches[4]) {
  if (!ctx) return PF_EINVAL;
  CU(cudaStreamSynchronize(ctx->stream));
  for (auto& e : ctx->graphs) graph_prof_collect(ctx, e);
  for (auto& o : ctx->ev_open) {
    float v = 0;
    cudaEventElapsedTime(&v, o.second.first, o.second.second);
    ctx->prof_ms[o.first] += v;
    ctx->prof_n[o.first] += 1;
    ctx->ev_pool.push_back(o.second.first);
    ctx->ev_pool.push_back(o.second.second);
  }
  ctx->ev_open.clear();
  for (int i = 0; i < 4; ++i) {
    if (ms) ms[i] = ctx->prof_ms[i];
    if (launches) launches[i] = ctx->nlaunch[i];
  }
  return PF_OK;
}

}  // extern "C"
