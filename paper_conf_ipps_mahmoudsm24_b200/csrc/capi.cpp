// capi.cpp — C ABI of liblbmr.so (include/lbmr.h) and the level scheduler.
//
// Scheduler (Algorithm 1, pipelined).  Level L runs 2^L substeps
// per coarse step.  F_L^k = the fused kernel that streams substep k
// of level L and collides substep k+1, writing C_L^{k+1} into buf[L][(k+1)%2].
// Driving the finest level k = 1, 2, ... and, after every F_L^k with k odd,
// running F_{L-1}^{(k+1)/2} recursively gives an order in which every read of
// Alg.1 sees the value it sees in the recursion:
//   same level C_L^k, Explosion C_{L-1}^{ceil(k/2)} (constant over the two fine
//   substeps, R-A4), Coalescence C_{L+1}^{2k-1} and C_{L+1}^{2k} (the two fine
//   post-collision states).
// 3 levels: F2^1 F1^1 F0^1 F2^2 F2^3 F1^2 F2^4 — 2^Lmax - 1 launches per
// coarse step, each moving 2Q values per leaf.  One coarse step is captured
// once into a CUDA graph per parity of the step index (level-0 buffers
// alternate) and replayed with cudaGraphLaunch.
#include <cuda_runtime.h>

#include <unistd.h>

#include <algorithm>
#include <bitset>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/lbmr.h"
#include "grid_builder.h"
#include "kernels.h"
#include "lattice.h"

using namespace lbmr;

namespace {

thread_local std::string g_err;

lbm_status fail(lbm_status s, const std::string& msg) {
  g_err = msg;
  return s;
}

#define CUDA_TRY(call)                                                                            \
  do {                                                                                            \
    cudaError_t e_ = (call);                                                                      \
    if (e_ != cudaSuccess) return fail(LBM_E_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

struct DevLevel {
  int32_t* blkmap = nullptr;
  uint8_t* types = nullptr;
  int32_t* origin = nullptr;
  int32_t* nbr = nullptr;
  int32_t* special_slot = nullptr;
  uint32_t* cellinfo = nullptr;
  uint32_t* bmask = nullptr;
  uint32_t* links = nullptr;
  uint32_t* coal = nullptr;
  int32_t* bpeer = nullptr;
  uint32_t* ghost_fill = nullptr;
  uint32_t* coal_fill = nullptr;
  uint32_t* coal_cand = nullptr;
  uint32_t* coal_wcand = nullptr;  // warp-cooperative gather units
  uint32_t* coal_wdst = nullptr;
  uint32_t* cg_qoff = nullptr;    // coalescence fused into the level kernel (product schedule)
  uint32_t* cg_cand = nullptr;
  uint32_t* cg_dest = nullptr;
  uint32_t* sc_qoff = nullptr;    // atomic Accumulate (ablation) scatter lists
  uint32_t* sc_items = nullptr;
  uint32_t* vfill = nullptr;   // volumetric variant lists (grid_builder.h)
  uint32_t* vavg = nullptr;
  void* vtemp = nullptr;
  void* pop[2] = {nullptr, nullptr};
  // neighbour rank on each side: its population buffers and the halo cell
  // index (in its grid) of every entry of our send list
  void* peer_pop[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};
  uint32_t* peer_cells[2] = {nullptr, nullptr};
};

}  // namespace

struct lbm_grid {
  lbm_grid_desc desc{};
  int levels = 0;
  int Q = 19;
  int coll = 0;
  int prec = 0;
  size_t tsize = 4;
  std::vector<HostLevel> host;
  std::vector<DevLevel> dev;
  std::vector<double> omega;
  BCEntry bc_host[256];
  BCEntry* bc_dev = nullptr;
  uint8_t face_host[27];
  uint8_t* face_dev = nullptr;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int device = 0;            // CUDA device the grid lives on (set by every call, restored after)
  // [par]: one coarse step starting at a step of parity par; [2 + par]: graph_steps
  // consecutive steps in one graph (fewer graph launches for short steps)
  cudaGraphExec_t graph[4] = {nullptr, nullptr, nullptr, nullptr};
  int graph_steps = 4;  // LBMR_GRAPH_STEPS; measured: cfg1 +13 % (fp32), +6.5 % (fp64), larger configs equal
  bool needs_prologue = true;
  bool init_locked = false;  // a step ran since the last init_uniform
  bool broken = false;
  int sched = LBM_SCHED_FUSED;  // lbm_set_schedule
  bool pdl = true;              // programmatic dependent launch of F_L^k after its gather (LBMR_NO_PDL=1: off)
  bool gather_warp = false;      // warp-cooperative gather kernel (LBMR_GATHER_WARP=1; default thread per entry)
  // L2 prefetch distance of the level kernels, in blocks (LBMR_PREFETCH; 0: off); re-swept
  // (profiles/r02_prefetch_resweep.txt): 64 vs 16 cfg5 fp32 +0.6 %, cfg4 KBC +0.4 %, Tab. I s3 +0.3 %
  int32_t prefetch = 64;
  bool peer_other_gpu[2] = {false, false};  // the connected neighbour on this side is on another GPU
  bool halo_spin = false;       // in-kernel halo waits (every connected neighbour on another GPU)
  bool nb_other_gpu = false;    // every connected neighbour is on another GPU (halo_spin without the env override)
  int64_t steps = 0;
  int64_t device_bytes = 0;
  std::vector<void*> allocs;
  // x-slab partition
  int n_ranks = 1, rank = 0;
  std::vector<int32_t> cuts;          // level-0 x cuts, n_ranks + 1 entries
  int32_t x_lo = 0;                   // global level-0 x of local x = 0
  int32_t has_nb[2] = {0, 0};
  bool connected[2] = {false, false};
  unsigned long long* flags = nullptr;      // [4], see kernels.h
  unsigned long long* peer_flags[2] = {nullptr, nullptr};
  std::vector<std::pair<std::string, void*>> ipc_open;  // opened IPC handles
  // reusable device / pinned host scratch of the diagnostics calls
  // (lbm_stats, lbm_probe): no allocation per call
  void* scratch = nullptr;
  size_t scratch_bytes = 0;
  void* hscratch = nullptr;
  size_t hscratch_bytes = 0;
};

namespace {

// Every call on a grid runs on the grid's device and restores the caller's
// current device afterwards (grids of one process may live on
// different devices).
struct DeviceGuard {
  int prev = -1;
  bool switched = false;
  explicit DeviceGuard(const lbm_grid* g) {
    if (g && cudaGetDevice(&prev) == cudaSuccess && prev != g->device)
      switched = cudaSetDevice(g->device) == cudaSuccess;
  }
  ~DeviceGuard() {
    if (switched) cudaSetDevice(prev);
  }
};

template <typename T>
lbm_status dev_upload(lbm_grid* g, T** dst, const std::vector<T>& src) {
  size_t bytes = std::max<size_t>(src.size() * sizeof(T), sizeof(T));
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) return fail(LBM_E_OOM, "cudaMalloc failed (tables)");
  g->allocs.push_back(p);
  g->device_bytes += (int64_t)bytes;
  // on the grid's stream and synchronised: a legacy-stream cudaMemcpy from
  // pageable memory may return before its DMA lands and is unordered with a
  // non-blocking user stream
  if (!src.empty()) {
    CUDA_TRY(cudaMemcpyAsync(p, src.data(), src.size() * sizeof(T), cudaMemcpyHostToDevice, g->stream));
    CUDA_TRY(cudaStreamSynchronize(g->stream));
  }
  *dst = static_cast<T*>(p);
  return LBM_OK;
}

lbm_status dev_alloc(lbm_grid* g, void** dst, size_t bytes) {
  bytes = std::max<size_t>(bytes, 16);
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) {
    cudaGetLastError();
    return fail(LBM_E_OOM, "cudaMalloc failed (" + std::to_string(bytes) + " bytes)");
  }
  g->allocs.push_back(p);
  g->device_bytes += (int64_t)bytes;
  *dst = p;
  return LBM_OK;
}

double omega_level(double omega0, int L) {
  // Eq.(9)
  const double p = std::ldexp(1.0, L);
  return 2.0 * omega0 / (2.0 * p + (1.0 - p) * omega0);
}

int bc_priority(int kind) { return kind == LBM_BC_VELOCITY ? 3 : kind == LBM_BC_NOSLIP ? 2 : 1; }

// face class per outside pattern (ox,oy,oz) in {-1,0,1}^3: VELOCITY > NOSLIP >
// OUTFLOW, ties to the first face in the order -x,+x,-y,+y,-z,+z (R-A11).
void compute_face_classes(lbm_grid* g) {
  for (int i = 0; i < 27; ++i) {
    int o[3] = {i % 3 - 1, (i / 3) % 3 - 1, i / 9 - 1};
    int best = g->desc.face_bc[0], bp = -1;
    for (int a = 0; a < 3; ++a) {
      if (!o[a]) continue;
      int cls = g->desc.face_bc[2 * a + (o[a] > 0 ? 1 : 0)];
      int pr = bc_priority(g->bc_host[cls].kind);
      if (pr > bp) { bp = pr; best = cls; }
    }
    g->face_host[i] = (uint8_t)best;
  }
}

size_t pop_bytes(const lbm_grid* g, int L) { return (size_t)g->host[L].nfluid * g->Q * kCells * g->tsize; }

LevelView view_of(const lbm_grid* g, int L) {
  LevelView v{};
  if (L < 0 || L >= g->levels) return v;
  const HostLevel& H = g->host[L];
  for (int a = 0; a < 3; ++a) { v.n[a] = (int32_t)H.n[a]; v.nb[a] = H.nb[a]; }
  v.blkmap = g->dev[L].blkmap;
  v.types = g->dev[L].types;
  return v;
}

template <typename T>
StepParams<T> make_params(const lbm_grid* g, int L, int64_t k) {
  StepParams<T> p{};
  const DevLevel& D = g->dev[L];
  p.own = view_of(g, L);
  p.coarse = view_of(g, L - 1);
  p.fine = view_of(g, L + 1);
  p.nbr = D.nbr;
  p.special_slot = D.special_slot;
  p.cellinfo = reinterpret_cast<const uint4*>(D.cellinfo);
  p.bmask = D.bmask;
  p.links = reinterpret_cast<const uint2*>(D.links);
  p.coal = D.coal;
  p.origin = D.origin;
  p.src = static_cast<const T*>(D.pop[k & 1]);
  p.dst = static_cast<T*>(D.pop[(k + 1) & 1]);
  if (L > 0) p.csrc = static_cast<const T*>(g->dev[L - 1].pop[((k + 1) / 2) & 1]);
  if (L + 1 < g->levels) {
    p.fa = static_cast<const T*>(g->dev[L + 1].pop[1]);  // C_{L+1}^{2k-1}
    p.fb = static_cast<const T*>(g->dev[L + 1].pop[0]);  // C_{L+1}^{2k}
  }
  p.bc = g->bc_dev;
  p.omega = (T)g->omega[L];
  p.prefetch = g->prefetch;
  for (int a = 0; a < 3; ++a) p.periodic[a] = g->desc.periodic[a];
  p.face_cls = g->face_dev;
  p.nfluid = g->host[L].nlaunch;
  p.ghost_fill = D.ghost_fill;
  p.nghost = (int32_t)(g->host[L].ghost_fill.size() / 3);
  p.vtemp = static_cast<const T*>(D.vtemp);
  if (g->desc.variant == LBM_VARIANT_VOLUMETRIC && L > 0 && ((k + 1) & 1) == 0) {
    // next substep is the second of the parent's substep: advected ghost packets
    p.nghost = 0;
    p.vfill = D.vfill;
    p.nvfill = (int32_t)(g->host[L].vfill.size() / 8);
  }
  if (L > 0) p.gsrc = static_cast<const T*>(g->dev[L - 1].pop[((k + 2) / 2) & 1]);  // C_{L-1}^{ceil((k+1)/2)}
  if (g->n_ranks > 1) {
    const HostLevel& H = g->host[L];
    p.nbctas = std::max(kHaloCtasPerBlock * H.nboundary, 1);
    p.halo_spin = g->halo_spin ? 1 : 0;
    p.nboundary = H.nboundary;
    p.flags = g->flags;
    p.bpeer = D.bpeer;
    for (int sd = 0; sd < 2; ++sd) {
      p.has_nb[sd] = g->has_nb[sd];
      if (!g->has_nb[sd]) continue;
      p.peer_flag[sd] = g->peer_flags[sd] + (1 - sd);  // we are the peer's neighbour on its other side
      p.peer_dst[sd] = static_cast<T*>(D.peer_pop[sd][(k + 1) & 1]);
      p.peer_cells[sd] = D.peer_cells[sd];
    }
  }
  return p;
}

// Schedule bits (lbmr.h LBM_SCHED_*), DESIGN.md §14:
//   UNFUSED    C and S of a level-substep as two kernels (S_L^k, in-place C)
//   SPLIT_E    Explosion as its own kernel E_L^k before S/F_L^k instead of the
//              trailing CTAs of the level's previous kernel
//   SPLIT_A    Accumulate as its own gather kernel after every fine Collision
//              (raw sums into the coarse ghost slots, initiated from the coarse
//              level: the paper's modified baseline)
//   ATOMIC_A   Accumulate as a scatter atomic write fused into the fine
//              Collision (CA fusion, Fig. 4c); the coarse kernel's
//              trailing CTAs reset the accumulators it no longer needs
//   SPLIT_O    Coalescence's division by 2|B| as its own kernel O_L^k before
//              the coarse S/F (otherwise fused: into the last gather, or
//              pre-scaled atomic terms)
//   CTA_GATHER A + A + O inside F_L^k: each CTA gathers its own cells'
//              coalescence links (no gather kernel)
// The product schedule (0) gathers A + A + O in one small warp-cooperative
// kernel right before F_L^k from the two retained fine buffers
// (deterministic, no atomics), F_L^k its programmatic dependent.
constexpr int kAblationBits =
    LBM_SCHED_SPLIT_E | LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A | LBM_SCHED_SPLIT_O | LBM_SCHED_CTA_GATHER;

// Coalescence inside F_L^k (CTA_GATHER): not with the unfused S kernel
// (256-thread CTAs), the split / atomic Accumulate or separate O.
bool fused_gather(int sched) {
  return (sched & LBM_SCHED_CTA_GATHER) &&
         !(sched & (LBM_SCHED_UNFUSED | LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A | LBM_SCHED_SPLIT_O));
}

bool level_has_coal(const lbm_grid* g, int L) {
  return L >= 0 && L + 1 < g->levels && !g->host[L].coal_fill.empty();
}

// Programmatic dependent launch of every kernel of the product schedule
// after the previous one (single rank, or ranks whose halo waits are
// in-kernel): a kernel's CTAs become resident during the previous kernel's
// tail instead of after its completion (LBMR_NO_PDL=1: off).  Not when a
// neighbour shares the GPU (in-kernel waits forced by LBMR_HALO_SPIN=1): the
// dependent grid's parked CTAs could then hold the SM slots the neighbour's
// kernel needs while our protocol CTAs spin for it.  On its own GPU a rank
// cannot starve itself: the dependent grid launches only once every CTA of
// the running kernel has started.
bool pdl_chain(const lbm_grid* g) {
  return g->pdl && !(g->sched & (LBM_SCHED_UNFUSED | (kAblationBits & ~LBM_SCHED_CTA_GATHER))) &&
         (g->n_ranks == 1 || (g->halo_spin && g->nb_other_gpu));
}

// The gather kernel reads L+1 halo cells of a partitioned grid: every CTA
// waits in-kernel when the neighbours are on other GPUs; otherwise a wait
// kernel precedes it (with in-kernel waits forced on a shared GPU, spinning
// gather CTAs could fill the SMs the neighbour's kernel needs).
bool gather_spins(const lbm_grid* g) { return g->n_ranks > 1 && g->halo_spin && g->nb_other_gpu; }

void launch_gather(lbm_grid* g, int L, const void* fa, const void* fb, void* dst, int mode, bool chain = false) {
  const HostLevel& H = g->host[L];
  const bool spin = gather_spins(g);
  if (g->gather_warp) {
    launch_coalesce_warp(g->prec, fa, fb, dst, g->dev[L].coal_wcand, g->dev[L].coal_wdst,
                         (int64_t)H.coal_wdst.size(), H.coal_wpair, mode, g->stream, spin ? g->flags : nullptr,
                         g->has_nb[0], g->has_nb[1], chain ? 1 : 0);
    return;
  }
  launch_coalesce(g->Q, g->prec, fa, fb, dst, g->dev[L].coal_fill, g->dev[L].coal_cand, H.coal_n[0], H.coal_n[1], mode,
                  g->stream, spin ? g->flags : nullptr, g->has_nb[0], g->has_nb[1], chain ? 1 : 0);
}

// In-kernel halo waits when every connected neighbour is on another GPU
// (LBMR_HALO_SPIN=1 / 0 forces them on / off).
void update_halo_spin(lbm_grid* g) {
  bool all = true;
  for (int sd = 0; sd < 2; ++sd)
    if (g->has_nb[sd] && !(g->connected[sd] && g->peer_other_gpu[sd])) all = false;
  // test hook: neighbours on SM-disjoint green contexts of one GPU behave like
  // neighbours on other GPUs (tests/test_gpu_green_partition.py)
  if (const char* e = getenv("LBMR_TEST_OTHER_GPU")) all = e[0] == '1';
  g->nb_other_gpu = all;
  if (const char* e = getenv("LBMR_HALO_SPIN")) all = e[0] == '1';
  g->halo_spin = all;
}

// ablation fields of the level-L launch producing C_L^{k+1} (k = 0: prologue)
template <typename T>
void ablation_params(lbm_grid* g, int L, int64_t k, StepParams<T>& p) {
  const int s = g->sched;
  if (s & LBM_SCHED_SPLIT_E) p.nghost = 0;
  if (s & LBM_SCHED_ATOMIC_A) {
    if (level_has_coal(g, L)) {  // reset the accumulators of dst (read by F_L^{k+1})
      p.zero_list = g->dev[L].coal_fill;
      p.nzero = (int32_t)g->host[L].coal_fill.size();
    }
    if (L > 0 && level_has_coal(g, L - 1) && !g->host[L].sc_items.empty()) {
      p.sc_qoff = g->dev[L].sc_qoff;
      p.sc_items = reinterpret_cast<const uint4*>(g->dev[L].sc_items);
      p.acc = static_cast<T*>(g->dev[L - 1].pop[((k + 2) / 2) & 1]);  // C_{L-1}^{ceil((k+1)/2)}'s buffer
      p.sc_scaled = (s & LBM_SCHED_SPLIT_O) ? 0 : 1;
    }
  }
}

// Explosion ghosts of C_L^k's buffer from C_{L-1}^{ceil(k/2)} (the E kernel)
template <typename T>
void refresh_ghosts(lbm_grid* g, int L, int64_t k) {
  StepParams<T> e = make_params<T>(g, L, k);
  e.dst = static_cast<T*>(g->dev[L].pop[k & 1]);
  e.gsrc = static_cast<const T*>(g->dev[L - 1].pop[((k + 1) / 2) & 1]);
  launch_level_step(g->Q, g->coll, g->prec, 5, &e, g->stream);
}

// SPLIT_A: after C_L^j was produced (j >= 1), accumulate it into the coarse
// ghost slots C_{L-1}^{ceil(j/2)} reads: the first fine substep sets the sum,
// the second adds (and divides unless SPLIT_O).
void accumulate_after(lbm_grid* g, int L, int64_t j) {
  if (!(g->sched & LBM_SCHED_SPLIT_A) || L == 0 || !level_has_coal(g, L - 1)) return;
  void* coarse = g->dev[L - 1].pop[((j + 1) / 2) & 1];
  const void* fine = g->dev[L].pop[j & 1];
  if (j & 1) launch_gather(g, L - 1, fine, nullptr, coarse, 0);
  else launch_gather(g, L - 1, nullptr, fine, coarse, kCoalFromDst | ((g->sched & LBM_SCHED_SPLIT_O) ? 0 : kCoalDivide));
}

// mid / mid_stamp (optional): an event recorded, or a timestamp written,
// after the pre-kernels (coalescence gather, volumetric averages, ablation
// kernels) and before the level kernel itself (per-level profiling)
template <typename T>
void launch_F_typed(lbm_grid* g, int L, int64_t k, int kind, cudaEvent_t mid = nullptr,
                    unsigned long long* mid_stamp = nullptr) {
  StepParams<T> p = make_params<T>(g, L, k);
  const int sched = g->sched;
  if (kind == 1) {  // prologue collision C_L^1
    ablation_params<T>(g, L, 0, p);
    if (sched & LBM_SCHED_SPLIT_E) p.nghost = (int32_t)(g->host[L].ghost_fill.size() / 3);  // initial ghosts
    launch_level_step(g->Q, g->coll, g->prec, 1, &p, g->stream);
    accumulate_after(g, L, 1);
    return;
  }
  const HostLevel& H = g->host[L];
  // volumetric variant: coarse averages of the children's arrivals into the
  // slots F_L^k pulls (gather, then scatter: DESIGN.md §16)
  if (!H.vavg.empty())
    launch_vavg(g->Q, g->prec, g->dev[L].vavg, (int32_t)(H.vavg.size() / 36), g->dev[L].pop[k & 1],
                g->dev[L + 1].pop[1], g->dev[L + 1].pop[0], g->bc_dev, g->face_dev, g->dev[L].vtemp, g->stream);
  // coalescence ghosts of C_L^k from C_{L+1}^{2k-1} and C_{L+1}^{2k} (both ready now)
  if (level_has_coal(g, L) && fused_gather(sched) && !g->host[L].cg_dest.empty()) {
    // CTA_GATHER: F_L^k's CTAs gather their own cells' links (no launch)
    p.cg_qoff = g->dev[L].cg_qoff;
    p.cg_cand = g->dev[L].cg_cand;
    p.cg_dest = g->dev[L].cg_dest;
  } else if (level_has_coal(g, L)) {
    if (g->n_ranks > 1 && !gather_spins(g)) {
      // the gather reads L+1 halo cells: it follows the neighbour wait of F_L^k,
      // which launch_level_step issues first; issue an explicit wait here instead
      launch_halo_wait(p.flags, p.has_nb[0], p.has_nb[1], g->stream);
    }
    void* dst = g->dev[L].pop[k & 1];
    if (!(sched & (LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A))) {
      launch_gather(g, L, g->dev[L + 1].pop[1], g->dev[L + 1].pop[0], dst,
                    (sched & LBM_SCHED_SPLIT_O) ? 0 : kCoalDivide, pdl_chain(g) && !mid_stamp);
      // the product schedule: F_L^k is the programmatic dependent of the
      // gather (its CTAs that do not pull coalescence ghosts overlap it)
      p.pdl = (g->n_ranks == 1 && !(sched & (LBM_SCHED_UNFUSED | kAblationBits)) && g->pdl) ? 1 : 0;
    }
    if (sched & LBM_SCHED_SPLIT_O) launch_gather(g, L, nullptr, nullptr, dst, kCoalFromDst | kCoalDivide);  // O
  }
  // E_L^k: refresh the ghosts of C_L^k's buffer from C_{L-1}^{ceil(k/2)}
  if ((sched & LBM_SCHED_SPLIT_E) && L > 0 && !H.ghost_fill.empty()) refresh_ghosts<T>(g, L, k);
  ablation_params<T>(g, L, k, p);
  if (mid) cudaEventRecord(mid, g->stream);
  if (mid_stamp) launch_stamp(mid_stamp, 0, g->stream);
  // the level kernel follows the previous kernel programmatically, unless a
  // halo wait kernel (ranks sharing a GPU) or a profiling stamp sits between
  p.pdl_chain = (pdl_chain(g) && !mid_stamp && !mid) ? 1 : 0;
  if (sched & LBM_SCHED_UNFUSED) {  // S_L^k then C_L^{k+1} in place (fusion ablation)
    StepParams<T> sp = p;  // the stream half: no scatter (nothing collided yet)
    sp.sc_qoff = nullptr;
    launch_level_step(g->Q, g->coll, g->prec, 3, &sp, g->stream);
    StepParams<T> c = p;
    c.src = p.dst;
    c.nghost = 0;
    c.nzero = 0;
    launch_level_step(g->Q, g->coll, g->prec, 4, &c, g->stream);
  } else {
    launch_level_step(g->Q, g->coll, g->prec, 0, &p, g->stream);
  }
  accumulate_after(g, L, k + 1);
}

void launch_F(lbm_grid* g, int L, int64_t k, int kind, cudaEvent_t mid = nullptr,
              unsigned long long* mid_stamp = nullptr) {
  if (g->prec == LBM_FP32) launch_F_typed<float>(g, L, k, kind, mid, mid_stamp);
  else launch_F_typed<double>(g, L, k, kind, mid, mid_stamp);
}

// The pipelined order of one coarse step n (0-based): list of (L, k).
void step_order(int levels, int64_t n, std::vector<std::pair<int, int64_t>>& out) {
  out.clear();
  const int F = levels - 1;
  const int64_t per = (int64_t)1 << F;
  for (int64_t k = per * n + 1; k <= per * (n + 1); ++k) {
    out.push_back({F, k});
    int L = F;
    int64_t kk = k;
    while (L > 0 && (kk & 1)) {
      kk = (kk + 1) / 2;
      --L;
      out.push_back({L, kk});
    }
  }
}

// Scratch buffers grow on demand; every user synchronises before returning,
// so a reallocation never races with work still reading the old buffer.
lbm_status scratch_dev(lbm_grid* g, size_t bytes, void** out) {
  if (g->scratch_bytes < bytes) {
    if (g->scratch) cudaFree(g->scratch);
    g->scratch = nullptr;
    g->scratch_bytes = 0;
    if (cudaMalloc(&g->scratch, bytes) != cudaSuccess) {
      cudaGetLastError();
      return fail(LBM_E_OOM, "cudaMalloc failed (scratch)");
    }
    g->scratch_bytes = bytes;
  }
  *out = g->scratch;
  return LBM_OK;
}

lbm_status scratch_host(lbm_grid* g, size_t bytes, void** out) {
  if (g->hscratch_bytes < bytes) {
    if (g->hscratch) cudaFreeHost(g->hscratch);
    g->hscratch = nullptr;
    g->hscratch_bytes = 0;
    if (cudaMallocHost(&g->hscratch, bytes) != cudaSuccess) {
      cudaGetLastError();
      return fail(LBM_E_OOM, "cudaMallocHost failed (scratch)");
    }
    g->hscratch_bytes = bytes;
  }
  *out = g->hscratch;
  return LBM_OK;
}

lbm_status run_prologue(lbm_grid* g) {
  // C_L^1 = Collision of the initial post-streaming state (buf 0 -> buf 1)
  for (int L = 0; L < g->levels; ++L) launch_F(g, L, 0, 1);
  CUDA_TRY(cudaGetLastError());
  g->needs_prologue = false;
  return LBM_OK;
}

lbm_status build_graphs(lbm_grid* g) {
  std::vector<std::pair<int, int64_t>> order, one;
  for (int gi = 0; gi < 4; ++gi) {
    const int par = gi & 1, nsteps = gi < 2 ? 1 : g->graph_steps;
    if (g->graph[gi] || (gi >= 2 && nsteps < 2)) continue;
    // a step's launches depend only on its parity (buffers alternate), so a
    // graph starting at parity par serves every start of that parity
    order.clear();
    for (int st = 0; st < nsteps; ++st) {
      step_order(g->levels, par + st, one);
      order.insert(order.end(), one.begin(), one.end());
    }
    cudaGraph_t graph;
    CUDA_TRY(cudaStreamBeginCapture(g->stream, cudaStreamCaptureModeThreadLocal));
    for (auto& lk : order) launch_F(g, lk.first, lk.second, 0);
    cudaError_t le = cudaGetLastError();
    CUDA_TRY(cudaStreamEndCapture(g->stream, &graph));
    if (le != cudaSuccess) return fail(LBM_E_CUDA, std::string("capture: ") + cudaGetErrorString(le));
    cudaError_t e = cudaGraphInstantiate(&g->graph[gi], graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) return fail(LBM_E_CUDA, std::string("cudaGraphInstantiate: ") + cudaGetErrorString(e));
    // upload now, so that its first launch does not pay for it
    CUDA_TRY(cudaGraphUpload(g->graph[gi], g->stream));
  }
  return LBM_OK;
}

int cur_buf(const lbm_grid* g, int L) {
  if (g->needs_prologue) return 0;
  // C_L^{k+1} with k = 2^L * steps
  const int64_t k = (g->steps << L);
  return (int)((k + 1) & 1);
}

}  // namespace

extern "C" {

const char* lbm_last_error(void) { return g_err.c_str(); }

const char* lbm_version(void) { return "lbmr 0.1 (sm_100a)"; }

int32_t lbm_schedule(int32_t levels, int64_t n, int64_t* order, int32_t capacity) {
  if (levels < 1 || levels > 16 || !order) return -1;
  std::vector<std::pair<int, int64_t>> o;
  step_order(levels, n, o);
  if ((int64_t)capacity < (int64_t)o.size()) return -1;
  for (size_t i = 0; i < o.size(); ++i) {
    order[2 * i] = o[i].first;
    order[2 * i + 1] = o[i].second;
  }
  return (int32_t)o.size();
}

int32_t lbm_lattice_table(int32_t Q, int32_t* e, double* w) {
  if ((Q != 19 && Q != 27) || !e || !w) return -1;
  for (int q = 0; q < Q; ++q) {
    e[3 * q] = kEx[q];
    e[3 * q + 1] = kEy[q];
    e[3 * q + 2] = kEz[q];
    w[q] = Q == 19 ? weight<19>(q) : weight<27>(q);
  }
  return Q;
}

double lbm_omega_level(double omega0, int32_t level) { return omega_level(omega0, level); }

static lbm_status validate_desc(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks) {
  if (!d || !masks) return fail(LBM_E_INVAL, "NULL argument");
  if (levels < 1 || levels > 16) return fail(LBM_E_INVAL, "levels must be in [1,16]");
  if (d->nx < 1 || d->ny < 1 || d->nz < 1) return fail(LBM_E_INVAL, "nx, ny, nz must be >= 1");
  for (int L = 0; L < levels; ++L)
    if (!masks[L]) return fail(LBM_E_INVAL, "masks[" + std::to_string(L) + "] is NULL");
  if (d->lattice != LBM_D3Q19 && d->lattice != LBM_D3Q27) return fail(LBM_E_INVAL, "lattice must be 19 or 27");
  if (d->collision != LBM_BGK && d->collision != LBM_KBC) return fail(LBM_E_INVAL, "bad collision");
  if (d->precision != LBM_FP32 && d->precision != LBM_FP64) return fail(LBM_E_INVAL, "bad precision");
  if (d->collision == LBM_KBC && d->lattice != LBM_D3Q27)
    return fail(LBM_E_UNSUPPORTED, "KBC requires D3Q27 (P:L260)");
  if (!(d->omega0 > 0.0 && d->omega0 < 2.0)) return fail(LBM_E_INVAL, "omega0 must be in (0, 2)");
  for (int a = 0; a < 3; ++a) {
    if (d->periodic[a]) continue;
    for (int s = 0; s < 2; ++s) {
      int c = d->face_bc[2 * a + s];
      if (c < 2 || c > 254) return fail(LBM_E_INVAL, "face_bc of a non-periodic face must be a BC class in 2..254");
    }
  }
  if (d->n_ranks < 1 || d->rank < 0 || d->rank >= d->n_ranks) return fail(LBM_E_INVAL, "bad n_ranks / rank");
  if (d->variant != LBM_VARIANT_PAPER && d->variant != LBM_VARIANT_VOLUMETRIC) return fail(LBM_E_INVAL, "bad variant");
  if (d->variant == LBM_VARIANT_VOLUMETRIC && d->n_ranks > 1)
    return fail(LBM_E_UNSUPPORTED, "the volumetric variant is single-rank only");
  if (d->n_ranks > d->nx) return fail(LBM_E_INVAL, "more ranks than level-0 x cells");
  for (int L = 0; L < levels; ++L) {
    int64_t n0 = (int64_t)d->nx << L, n1 = (int64_t)d->ny << L, n2 = (int64_t)d->nz << L;
    if (n0 > (1 << 28) || n1 > (1 << 28) || n2 > (1 << 28)) return fail(LBM_E_INVAL, "level too large");
  }
  return LBM_OK;
}

// Balanced x-slab cuts at coarse-cell boundaries: the work of
// level-0 column x is sum_L 2^L * (fluid leaves of level L inside it).
static void partition_cuts(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks, int P,
                           std::vector<int32_t>& cuts) {
  const int nx = d->nx;
  std::vector<double> W(nx, 0.0);
  for (int L = 0; L < levels; ++L) {
    const int64_t plane = ((int64_t)d->ny << L) * ((int64_t)d->nz << L);
    const int64_t nxl = (int64_t)nx << L;
    std::vector<int64_t> cnt(nxl, 0);
#pragma omp parallel for schedule(static)
    for (int64_t x = 0; x < nxl; ++x) {
      const uint8_t* m = masks[L] + x * plane;
      int64_t c = 0;
      for (int64_t i = 0; i < plane; ++i) c += (m[i] == 1);
      cnt[x] = c;
    }
    for (int64_t x = 0; x < nxl; ++x) W[x >> L] += (double)(cnt[x] << L);
  }
  std::vector<double> pre(nx + 1, 0.0);
  for (int x = 0; x < nx; ++x) pre[x + 1] = pre[x] + W[x];
  cuts.assign(P + 1, 0);
  cuts[P] = nx;
  for (int r = 1; r < P; ++r) {
    const double target = pre[nx] * r / P;
    int x = (int)(std::lower_bound(pre.begin(), pre.end(), target) - pre.begin());
    if (x > 0 && target - pre[x - 1] < pre[x] - target) --x;
    x = std::max(x, cuts[r - 1] + 1);
    x = std::min(x, nx - (P - r));
    cuts[r] = x;
  }
}

struct LocalSlab {
  lbm_grid_desc desc;                      // local dims, x non-periodic
  std::vector<std::vector<uint8_t>> masks; // local masks (slab + halo)
  std::vector<const uint8_t*> ptrs;
  int32_t x_lo = 0, owned_lo0 = 0, owned_hi0 = -1, has_nb[2] = {0, 0};
};

static void make_local(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks,
                       const std::vector<int32_t>& cuts, LocalSlab& out) {
  const int P = d->n_ranks, r = d->rank;
  const bool per = d->periodic[0] != 0;
  out.has_nb[0] = (r > 0 || per) ? 1 : 0;
  out.has_nb[1] = (r < P - 1 || per) ? 1 : 0;
  out.x_lo = cuts[r] - out.has_nb[0];
  const int x_hi = cuts[r + 1] + out.has_nb[1];
  const int nxl = x_hi - out.x_lo;
  out.desc = *d;
  out.desc.nx = nxl;
  out.desc.periodic[0] = 0;
  out.owned_lo0 = out.has_nb[0];
  out.owned_hi0 = nxl - out.has_nb[1];
  out.masks.resize(levels);
  for (int L = 0; L < levels; ++L) {
    const int64_t plane = ((int64_t)d->ny << L) * ((int64_t)d->nz << L);
    const int64_t gn = (int64_t)d->nx << L, ln = (int64_t)nxl << L;
    out.masks[L].resize(ln * plane);
    for (int64_t x = 0; x < ln; ++x) {
      const int64_t gx = (((int64_t)out.x_lo << L) + x + gn) % gn;
      std::memcpy(&out.masks[L][x * plane], masks[L] + gx * plane, plane);
    }
    out.ptrs.push_back(out.masks[L].data());
  }
}

static lbm_status build_host(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks,
                             std::vector<HostLevel>& host, LocalSlab* slab = nullptr) {
  BuildInput in{};
  in.n0[0] = d->nx; in.n0[1] = d->ny; in.n0[2] = d->nz;
  for (int a = 0; a < 3; ++a) in.periodic[a] = d->periodic[a] ? 1 : 0;
  in.levels = levels;
  in.Q = d->lattice;
  in.masks = masks;
  in.variant = d->variant;
  in.align_blocks = getenv("LBMR_NO_BLOCK_ALIGN") ? 0 : 1;  // A/B switch for measurements
  if (const char* o = getenv("LBMR_BLOCK_ORDER"))
    in.block_order = std::strcmp(o, "raster") == 0 ? 1 : std::strcmp(o, "hilbert") == 0 ? 2 : 0;
  if (slab) {
    in.n0[0] = slab->desc.nx;
    in.periodic[0] = 0;
    in.masks = slab->ptrs.data();
    in.owned_lo0 = slab->owned_lo0;
    in.owned_hi0 = slab->owned_hi0;
    in.has_nb[0] = slab->has_nb[0];
    in.has_nb[1] = slab->has_nb[1];
  }
  std::string err;
  int st = build_grid(in, host, err);
  if (st) return fail((lbm_status)st, err);
  for (int L = 0; L < levels; ++L)
    if ((uint64_t)host[L].nblocks * (uint64_t)d->lattice * kCells >= (1ull << 32))
      return fail(LBM_E_UNSUPPORTED, "level " + std::to_string(L) +
                                         " too large for one device (> 2^32 populations); use more ranks");
  return LBM_OK;
}

// Device bytes lbm_grid_create allocates for these host tables: the same list
// (and the same minimum sizes) as its dev_upload / dev_alloc calls.
static int64_t planned_device_bytes(const std::vector<HostLevel>& host, int Q, size_t ts, int n_ranks) {
  auto up = [](size_t n, size_t es) { return (int64_t)std::max(n * es, es); };
  auto al = [](size_t b) { return (int64_t)std::max<size_t>(b, 16); };
  int64_t t = 0;
  for (const HostLevel& H : host)
    t += up(H.blkmap.size(), 4) + up(H.types.size(), 1) + up(H.origin.size(), 4) + up(H.nbr.size(), 4) +
         up(H.special_slot.size(), 4) + up(H.cellinfo.size(), 4) + up(H.bmask.size(), 4) + up(H.links.size(), 4) +
         up(H.coal.size(), 4) + up(H.bpeer.size(), 4) + up(H.ghost_fill.size(), 4) + up(H.coal_fill.size(), 4) +
         up(H.coal_cand.size(), 4) + up(H.coal_wcand.size(), 4) + up(H.coal_wdst.size(), 4) + up(H.cg_qoff.size(), 4) + up(H.cg_cand.size(), 4) + up(H.cg_dest.size(), 4) +
         up(H.sc_qoff.size(), 4) + up(H.sc_items.size(), 4) + up(H.vfill.size(), 4) +
         up(H.vavg.size(), 4) + al((H.vavg.size() / 36) * ts) +
         2 * al((size_t)H.nfluid * Q * kCells * ts);
  if (n_ranks > 1) t += al(4 * sizeof(unsigned long long));
  t += al(sizeof(BCEntry) * 256) + al(32);
  return t;
}

static void fill_info(const std::vector<HostLevel>& host, int Q, int prec, int n_ranks, lbm_grid_info* info,
                      int sched = 0, bool halo_spin = false, bool gather_spin = false) {
  std::memset(info, 0, sizeof(*info));
  info->levels = (int32_t)host.size();
  info->Q = Q;
  info->precision = prec;
  info->kernels_per_step = (1 << host.size()) - 1;
  info->launches_per_step = info->kernels_per_step;
  // partitioned grid: a one-thread halo wait before every level kernel
  // (unless the waits are in-kernel: neighbours on other GPUs)
  const bool waits = n_ranks > 1 && !halo_spin;
  if (waits) info->launches_per_step += info->kernels_per_step;
  for (size_t L = 0; L < host.size(); ++L) {
    // the coalescence gather before every F_L^k (and its own halo wait when
    // partitioned), unless fused into F_L^k (product)
    const bool gather_waits = n_ranks > 1 && !gather_spin;
    if (!host[L].coal_fill.empty() && !fused_gather(sched))
      info->launches_per_step += ((int64_t)1 << L) * (gather_waits ? 2 : 1);
    if (!host[L].vavg.empty()) info->launches_per_step += (int64_t)2 << L;
    // ablation schedules (lbm_set_schedule): split kernels per level-substep
    const int64_t sub = (int64_t)1 << L;
    const bool coal = L + 1 < (int)host.size() && !host[L].coal_fill.empty();
    if (sched & LBM_SCHED_UNFUSED) info->launches_per_step += sub;  // S and C
    if (coal && (sched & (LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A))) info->launches_per_step -= sub;  // no gather
    if (coal && (sched & LBM_SCHED_SPLIT_A)) info->launches_per_step += sub * 2;  // A after each fine substep
    if (coal && (sched & LBM_SCHED_SPLIT_O)) info->launches_per_step += sub;  // O
    if ((sched & LBM_SCHED_SPLIT_E) && L > 0 && !host[L].ghost_fill.empty()) info->launches_per_step += sub;  // E
    info->leaves[L] = host[L].leaves;
    for (int a = 0; a < 3; ++a) info->block_offset[L][a] = host[L].off[a];
    info->blocks[L] = host[L].nfluid;
    info->special_blocks[L] = host[L].nspecial;
    info->special_cells[L] = host[L].special_cells;
    info->total_blocks[L] = host[L].nblocks;
    info->coal_links[L] = host[L].coal_n[0] + host[L].coal_n[1];
    info->coal_wide[L] = host[L].coal_n[1];
  }
}

lbm_status lbm_grid_analyze(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks,
                            lbm_grid_info* info) {
  g_err.clear();
  if (!info) return fail(LBM_E_INVAL, "NULL info");
  lbm_status s = validate_desc(d, levels, masks);
  if (s) return s;
  std::vector<HostLevel> host;
  if (d->n_ranks > 1) {
    std::vector<int32_t> cuts;
    partition_cuts(d, levels, masks, d->n_ranks, cuts);
    LocalSlab slab;
    make_local(d, levels, masks, cuts, slab);
    if ((s = build_host(d, levels, masks, host, &slab))) return s;
  } else if ((s = build_host(d, levels, masks, host))) {
    return s;
  }
  fill_info(host, d->lattice, d->precision, d->n_ranks, info);
  info->device_bytes = planned_device_bytes(host, d->lattice, d->precision == LBM_FP32 ? 4 : 8, d->n_ranks);
  return LBM_OK;
}

lbm_status lbm_grid_create(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks, lbm_grid** out) {
  g_err.clear();
  if (!out) return fail(LBM_E_INVAL, "NULL argument");
  *out = nullptr;
  lbm_status vs = validate_desc(d, levels, masks);
  if (vs) return vs;

  lbm_grid* g = new lbm_grid();
  g->desc = *d;
  g->levels = levels;
  g->Q = d->lattice;
  g->coll = d->collision;
  g->prec = d->precision;
  g->tsize = d->precision == LBM_FP32 ? 4 : 8;
  g->pdl = getenv("LBMR_NO_PDL") == nullptr;
  if (const char* e = getenv("LBMR_GATHER_WARP")) g->gather_warp = e[0] != '0';
  if (const char* e = getenv("LBMR_GRAPH_STEPS")) g->graph_steps = std::max(1, std::min(64, atoi(e)));
  if (const char* e = getenv("LBMR_PREFETCH")) g->prefetch = std::max(0, atoi(e));
  for (int c = 0; c < 256; ++c) {
    g->bc_host[c].kind = LBM_BC_NOSLIP;
    g->bc_host[c].pad_ = 0;
    g->bc_host[c].u[0] = g->bc_host[c].u[1] = g->bc_host[c].u[2] = 0.0;
  }
  g->n_ranks = d->n_ranks;
  g->rank = d->rank;
  if (d->n_ranks > 1) {
    partition_cuts(d, levels, masks, d->n_ranks, g->cuts);
    LocalSlab slab;
    make_local(d, levels, masks, g->cuts, slab);
    g->x_lo = slab.x_lo;
    g->has_nb[0] = slab.has_nb[0];
    g->has_nb[1] = slab.has_nb[1];
    vs = build_host(d, levels, masks, g->host, &slab);
  } else {
    g->cuts = {0, d->nx};
    vs = build_host(d, levels, masks, g->host);
  }
  if (vs) {
    delete g;
    return vs;
  }
  for (int L = 0; L < levels; ++L) g->omega.push_back(omega_level(d->omega0, L));

  auto cleanup = [&](lbm_status s) {
    std::string keep = g_err;
    lbm_grid_destroy(g);
    g_err = keep;
    return s;
  };
  if (cudaGetDevice(&g->device) != cudaSuccess) {
    delete g;
    return fail(LBM_E_CUDA, "cudaGetDevice failed (no CUDA device?)");
  }
  if (d->stream) {
    g->stream = static_cast<cudaStream_t>(d->stream);
  } else {
    if (cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking) != cudaSuccess) {
      delete g;
      return fail(LBM_E_CUDA, "cudaStreamCreate failed (no CUDA device?)");
    }
    g->own_stream = true;
  }

  // eager kernel loading, once per device (the function attributes and the
  // module load are per device; guarded for grids created from several threads)
  {
    static std::mutex mu;
    static std::bitset<64> preloaded;
    std::lock_guard<std::mutex> lock(mu);
    if (g->device >= 0 && g->device < 64 && !preloaded[g->device]) {
      preload_kernels();
      preloaded[g->device] = true;
    }
  }
  g->dev.resize(levels);
  lbm_status s;
  for (int L = 0; L < levels; ++L) {
    HostLevel& H = g->host[L];
    DevLevel& D = g->dev[L];
    if ((s = dev_upload(g, &D.blkmap, H.blkmap))) return cleanup(s);
    if ((s = dev_upload(g, &D.types, H.types))) return cleanup(s);
    if ((s = dev_upload(g, &D.origin, H.origin))) return cleanup(s);
    if ((s = dev_upload(g, &D.nbr, H.nbr))) return cleanup(s);
    if ((s = dev_upload(g, &D.special_slot, H.special_slot))) return cleanup(s);
    if ((s = dev_upload(g, &D.cellinfo, H.cellinfo))) return cleanup(s);
    if ((s = dev_upload(g, &D.bmask, H.bmask))) return cleanup(s);
    if ((s = dev_upload(g, &D.links, H.links))) return cleanup(s);
    if ((s = dev_upload(g, &D.coal, H.coal))) return cleanup(s);
    if ((s = dev_upload(g, &D.bpeer, H.bpeer))) return cleanup(s);
    if ((s = dev_upload(g, &D.ghost_fill, H.ghost_fill))) return cleanup(s);
    if ((s = dev_upload(g, &D.coal_fill, H.coal_fill))) return cleanup(s);
    if ((s = dev_upload(g, &D.coal_cand, H.coal_cand))) return cleanup(s);
    if ((s = dev_upload(g, &D.coal_wcand, H.coal_wcand))) return cleanup(s);
    if ((s = dev_upload(g, &D.coal_wdst, H.coal_wdst))) return cleanup(s);
    if ((s = dev_upload(g, &D.cg_qoff, H.cg_qoff))) return cleanup(s);
    if ((s = dev_upload(g, &D.cg_cand, H.cg_cand))) return cleanup(s);
    if ((s = dev_upload(g, &D.cg_dest, H.cg_dest))) return cleanup(s);
    if ((s = dev_upload(g, &D.sc_qoff, H.sc_qoff))) return cleanup(s);
    if ((s = dev_upload(g, &D.sc_items, H.sc_items))) return cleanup(s);
    if ((s = dev_upload(g, &D.vfill, H.vfill))) return cleanup(s);
    if ((s = dev_upload(g, &D.vavg, H.vavg))) return cleanup(s);
    if ((s = dev_alloc(g, &D.vtemp, (H.vavg.size() / 36) * g->tsize))) return cleanup(s);
    for (int b = 0; b < 2; ++b) {
      if ((s = dev_alloc(g, &D.pop[b], pop_bytes(g, L)))) return cleanup(s);
      // on the grid's stream: a legacy-stream memset is unordered with a
      // non-blocking user stream and could land after the first halo stores
      if (cudaMemsetAsync(D.pop[b], 0, pop_bytes(g, L), g->stream) != cudaSuccess)
        return cleanup(fail(LBM_E_CUDA, "memset"));
    }
    // the dense per-level tables are on the device now; keep only counters
    // (the host block map is kept for lbm_probe)
    std::vector<uint32_t>().swap(H.cellinfo);
    std::vector<uint32_t>().swap(H.bmask);
    std::vector<uint32_t>().swap(H.links);
    std::vector<uint32_t>().swap(H.coal);
    std::vector<int32_t>().swap(H.nbr);
    std::vector<uint8_t>().swap(H.ghost);
  }
  void* p;
  if (g->n_ranks > 1) {  // halo-protocol flags, own allocation so it can be shared by CUDA IPC
    if ((s = dev_alloc(g, &p, 4 * sizeof(unsigned long long)))) return cleanup(s);
    if (cudaMemsetAsync(p, 0, 4 * sizeof(unsigned long long), g->stream) != cudaSuccess)
      return cleanup(fail(LBM_E_CUDA, "memset"));
    g->flags = static_cast<unsigned long long*>(p);
  }
  if ((s = dev_alloc(g, &p, sizeof(BCEntry) * 256))) return cleanup(s);
  g->bc_dev = static_cast<BCEntry*>(p);
  if ((s = dev_alloc(g, &p, 32))) return cleanup(s);
  g->face_dev = static_cast<uint8_t*>(p);
  compute_face_classes(g);
  // same stream as lbm_set_bc's updates: a legacy-stream copy here could land
  // after them (pageable cudaMemcpy returns before its DMA completes) and
  // restore the default edge/corner classes (seen as a missing moving-wall
  // term on lid edges in rare two-process runs)
  if (cudaMemcpyAsync(g->bc_dev, g->bc_host, sizeof(g->bc_host), cudaMemcpyHostToDevice, g->stream) != cudaSuccess ||
      cudaMemcpyAsync(g->face_dev, g->face_host, 27, cudaMemcpyHostToDevice, g->stream) != cudaSuccess)
    return cleanup(fail(LBM_E_CUDA, "upload BC table"));
  if (cudaStreamSynchronize(g->stream) != cudaSuccess) return cleanup(fail(LBM_E_CUDA, "zero-fill"));
  // populations start as g = 0, i.e. f = w (rest equilibrium, rho = 1)
  g->needs_prologue = true;
  *out = g;
  return LBM_OK;
}

lbm_status lbm_set_bc(lbm_grid* g, int32_t cls, int32_t kind, const double* u) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (cls < 2 || cls > 254) return fail(LBM_E_INVAL, "bc_class must be in 2..254");
  if (kind != LBM_BC_NOSLIP && kind != LBM_BC_VELOCITY && kind != LBM_BC_OUTFLOW)
    return fail(LBM_E_INVAL, "bad BC kind");
  g->bc_host[cls].kind = kind;
  for (int a = 0; a < 3; ++a) g->bc_host[cls].u[a] = u ? u[a] : 0.0;
  compute_face_classes(g);
  FaceTable ft{};
  std::memcpy(ft.cls, g->face_host, 27);
  launch_bc_update(g->bc_dev, cls, g->bc_host[cls], g->face_dev, ft, g->stream);
  CUDA_TRY(cudaGetLastError());
  return LBM_OK;
}

// Host -> device traffic of the init / output calls goes through the grid's
// reusable pinned host and device scratch (no allocation per call), in chunks
// of kIoChunkBlocks blocks so the scratch stays small (64 MiB) at any size.
constexpr int32_t kIoChunkBlocks = 4096;

static lbm_status init_level(lbm_grid* g, int L, const double* rho, const double* u, double rho0, const double* u0) {
  const HostLevel& H = g->host[L];
  const size_t chunk_cells = (size_t)kIoChunkBlocks * kCells;
  void *dv = nullptr, *hv = nullptr;
  lbm_status st;
  CUDA_TRY(cudaStreamSynchronize(g->stream));  // queued work may still read the scratch
  if ((st = scratch_dev(g, chunk_cells * 4 * sizeof(double), &dv)) ||
      (st = scratch_host(g, chunk_cells * 4 * sizeof(double), &hv)))
    return st;
  for (int32_t b0 = 0; b0 < H.nfluid; b0 += kIoChunkBlocks) {
    const int32_t nb = std::min(kIoChunkBlocks, H.nfluid - b0);
    const size_t ncell = (size_t)nb * kCells;
    // chunk layout: rho[ncell] then u[3 ncell]
    double* r = static_cast<double*>(hv);
    double* v = r + ncell;
#pragma omp parallel for schedule(static)
    for (int32_t i = 0; i < nb; ++i) {
      const int32_t b = b0 + i;
      for (int l = 0; l < kCells; ++l) {
        const size_t k = (size_t)i * kCells + l;
        r[k] = rho0;
        v[3 * k] = u0 ? u0[0] : 0.0;
        v[3 * k + 1] = u0 ? u0[1] : 0.0;
        v[3 * k + 2] = u0 ? u0[2] : 0.0;
        if (!(rho || u) || H.types[(size_t)b * kCells + l] != kFluid) continue;
        const int64_t x = H.cell_x(b, l), y = H.cell_y(b, l), z = H.cell_z(b, l);
        if (x < H.owned_lo || x >= H.owned_hi) continue;  // halo cells come from the neighbour
        const int64_t c = ((x - H.owned_lo) * H.n[1] + y) * H.n[2] + z;
        if (rho) r[k] = rho[c];
        if (u) { v[3 * k] = u[3 * c]; v[3 * k + 1] = u[3 * c + 1]; v[3 * k + 2] = u[3 * c + 2]; }
      }
    }
    double* dr = static_cast<double*>(dv);
    CUDA_TRY(cudaMemcpyAsync(dr, r, ncell * 4 * sizeof(double), cudaMemcpyHostToDevice, g->stream));
    launch_init_eq(g->Q, g->prec, static_cast<char*>(g->dev[L].pop[0]) + (size_t)b0 * g->Q * kCells * g->tsize,
                   g->dev[L].types + (size_t)b0 * kCells, nb, dr, dr + ncell, g->stream);
    CUDA_TRY(cudaGetLastError());
    CUDA_TRY(cudaStreamSynchronize(g->stream));  // the pinned chunk is refilled next
  }
  return LBM_OK;
}

lbm_status lbm_init_equilibrium(lbm_grid* g, int32_t level, const double* rho, const double* u) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (g->broken) return fail(LBM_E_STATE, "grid is in an error state");
  if (level < 0 || level >= g->levels) return fail(LBM_E_INVAL, "level out of range");
  if (g->init_locked)
    return fail(LBM_E_STATE, "lbm_init_equilibrium after lbm_step: call lbm_init_uniform first");
  lbm_status s = init_level(g, level, rho, u, 1.0, nullptr);
  if (s) return s;
  g->needs_prologue = true;
  g->steps = 0;
  return LBM_OK;
}

lbm_status lbm_init_uniform(lbm_grid* g, double rho0, const double* u0) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (g->broken) return fail(LBM_E_STATE, "grid is in an error state");
  for (int L = 0; L < g->levels; ++L) {
    lbm_status s = init_level(g, L, nullptr, nullptr, rho0, u0);
    if (s) return s;
  }
  g->needs_prologue = true;
  g->init_locked = false;
  g->steps = 0;
  return LBM_OK;
}

lbm_status lbm_step(lbm_grid* g, int32_t n) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (g->broken) return fail(LBM_E_STATE, "grid is in an error state");
  if (n < 0) return fail(LBM_E_INVAL, "n_coarse must be >= 0");
  if (n == 0) return LBM_OK;
  for (int sd = 0; sd < 2; ++sd)
    if (g->n_ranks > 1 && g->has_nb[sd] && !g->connected[sd])
      return fail(LBM_E_STATE, "halo side " + std::to_string(sd) + " not connected");
  lbm_status s;
  if (g->needs_prologue && (s = run_prologue(g))) { g->broken = true; return s; }
  if (getenv("LBMR_DEBUG_PROLOGUE_ONLY")) return LBM_OK;
  if ((g->sched & LBM_SCHED_NO_GRAPH) || getenv("LBMR_DEBUG_NO_GRAPH")) {
    std::vector<std::pair<int, int64_t>> order;
    for (int i = 0; i < n; ++i) {
      step_order(g->levels, g->steps, order);
      for (auto& lk : order) launch_F(g, lk.first, lk.second, 0);
      ++g->steps;
    }
    g->init_locked = true;
    return LBM_OK;
  }
  if ((s = build_graphs(g))) { g->broken = true; return s; }
  while (n > 0) {
    const bool multi = g->graph_steps > 1 && n >= g->graph_steps;
    cudaError_t e = cudaGraphLaunch(g->graph[(multi ? 2 : 0) + (g->steps & 1)], g->stream);
    if (e != cudaSuccess) {
      g->broken = true;
      return fail(LBM_E_CUDA, std::string("cudaGraphLaunch: ") + cudaGetErrorString(e));
    }
    g->steps += multi ? g->graph_steps : 1;
    n -= multi ? g->graph_steps : 1;
  }
  g->init_locked = true;
  return LBM_OK;
}

lbm_status lbm_set_schedule(lbm_grid* g, int32_t mode) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  const int all = LBM_SCHED_UNFUSED | LBM_SCHED_NO_GRAPH | kAblationBits;
  if (mode < 0 || (mode & ~all)) return fail(LBM_E_INVAL, "bad schedule mode");
  if ((mode & (LBM_SCHED_UNFUSED | kAblationBits)) && g->n_ranks > 1)
    return fail(LBM_E_UNSUPPORTED, "the ablation schedules are single-rank only");
  if ((mode & kAblationBits) && g->desc.variant != LBM_VARIANT_PAPER)
    return fail(LBM_E_UNSUPPORTED, "the E/A/O ablation schedules need the paper variant");
  if ((mode & LBM_SCHED_SPLIT_A) && (mode & LBM_SCHED_ATOMIC_A))
    return fail(LBM_E_INVAL, "SPLIT_A and ATOMIC_A are two forms of the same Accumulate: choose one");
  if (mode == g->sched) return LBM_OK;
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  for (int p = 0; p < 4; ++p)
    if (g->graph[p]) {
      cudaGraphExecDestroy(g->graph[p]);
      g->graph[p] = nullptr;
    }
  const int acc_old = g->sched & (LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A | LBM_SCHED_SPLIT_O);
  const bool leave_split_e = (g->sched & LBM_SCHED_SPLIT_E) && !(mode & LBM_SCHED_SPLIT_E);
  g->sched = mode;
  if (!g->needs_prologue && leave_split_e) {
    // under SPLIT_E the explosion ghosts of the current buffers are refreshed
    // by the E kernel right before they are read; the fused kernels expect the
    // previous kernel to have done it: refresh them now
    for (int L = 1; L < g->levels; ++L) {
      if (g->host[L].ghost_fill.empty()) continue;
      const int64_t k = (g->steps << L) + 1;  // next substep of level L
      if (g->prec == LBM_FP32) refresh_ghosts<float>(g, L, k);
      else refresh_ghosts<double>(g, L, k);
    }
    CUDA_TRY(cudaGetLastError());
  }
  const int acc_new = mode & (LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A | LBM_SCHED_SPLIT_O);
  if (!g->needs_prologue && acc_new != acc_old && (mode & (LBM_SCHED_SPLIT_A | LBM_SCHED_ATOMIC_A))) {
    // At a coarse-step boundary the first fine substep of every coarse
    // level's next substep has run already: its accumulation (kept implicitly
    // in the fine buffer by the product schedule) is rebuilt in the form the
    // new schedule expects in the coarse ghost slots.
    for (int L = 0; L + 1 < g->levels; ++L) {
      if (!level_has_coal(g, L)) continue;
      const int64_t k = (g->steps << L) + 1;  // next substep of level L
      const bool pre_scaled = (mode & LBM_SCHED_ATOMIC_A) && !(mode & LBM_SCHED_SPLIT_O);
      launch_gather(g, L, g->dev[L + 1].pop[1], nullptr, g->dev[L].pop[k & 1], pre_scaled ? kCoalDivide : 0);
    }
    CUDA_TRY(cudaGetLastError());
    CUDA_TRY(cudaStreamSynchronize(g->stream));
  }
  return LBM_OK;
}

// ---- checkpoint / resume --------------------------------------------------
// Layout: CkptHeader, then per level the current population buffer
// (post-collision state C_L^{k+1} incl. its explosion/coalescence ghosts, or
// the initial post-streaming state before the first step).  At a coarse-step
// boundary nothing else is live: every other buffer is rewritten before it is
// read in the next step, which the resume tests check bitwise.
namespace {
struct CkptHeader {
  uint32_t magic, version;
  int32_t levels, Q, coll, prec, n_ranks, rank;
  int64_t steps;
  int32_t needs_prologue, sched;
  int64_t nfluid[16];
  int64_t leaves[16];
};
constexpr uint32_t kCkptMagic = 0x4b434d4cu;  // "LMCK"
}  // namespace

lbm_status lbm_checkpoint_size(const lbm_grid* g, int64_t* bytes) {
  g_err.clear();
  if (!g || !bytes) return fail(LBM_E_INVAL, "NULL argument");
  int64_t n = sizeof(CkptHeader);
  for (int L = 0; L < g->levels; ++L) n += (int64_t)pop_bytes(g, L);
  *bytes = n;
  return LBM_OK;
}

lbm_status lbm_checkpoint_save(lbm_grid* g, void* host, int64_t capacity) {
  g_err.clear();
  if (!g || !host) return fail(LBM_E_INVAL, "NULL argument");
  DeviceGuard dg_(g);
  if (g->broken) return fail(LBM_E_STATE, "grid is in an error state");
  int64_t need = 0;
  lbm_checkpoint_size(g, &need);
  if (capacity < need) return fail(LBM_E_INVAL, "checkpoint buffer too small");
  CkptHeader h;
  std::memset(&h, 0, sizeof(h));
  h.magic = kCkptMagic;
  h.version = 1;
  h.levels = g->levels;
  h.Q = g->Q;
  h.coll = g->coll;
  h.prec = g->prec;
  h.n_ranks = g->n_ranks;
  h.rank = g->rank;
  h.steps = g->steps;
  h.needs_prologue = g->needs_prologue ? 1 : 0;
  h.sched = g->sched;
  for (int L = 0; L < g->levels; ++L) {
    h.nfluid[L] = g->host[L].nfluid;
    h.leaves[L] = g->host[L].leaves;
  }
  char* out = static_cast<char*>(host);
  std::memcpy(out, &h, sizeof(h));
  int64_t off = sizeof(h);
  // partitioned grid: the buffers include halo cells the neighbours' last
  // kernels store into; wait (on the device) until every neighbour has
  // finished the cut-plane part of all kernels this rank has run
  if (g->n_ranks > 1 && !g->needs_prologue) launch_halo_wait(g->flags, g->has_nb[0], g->has_nb[1], g->stream);
  CUDA_TRY(cudaGetLastError());
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  for (int L = 0; L < g->levels; ++L) {
    const size_t b = pop_bytes(g, L);
    CUDA_TRY(cudaMemcpyAsync(out + off, g->dev[L].pop[cur_buf(g, L)], b, cudaMemcpyDeviceToHost, g->stream));
    off += (int64_t)b;
  }
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  return LBM_OK;
}

lbm_status lbm_checkpoint_load(lbm_grid* g, const void* host, int64_t size) {
  g_err.clear();
  if (!g || !host) return fail(LBM_E_INVAL, "NULL argument");
  DeviceGuard dg_(g);
  if (g->broken) return fail(LBM_E_STATE, "grid is in an error state");
  if (size < (int64_t)sizeof(CkptHeader)) return fail(LBM_E_INVAL, "checkpoint too small");
  CkptHeader h;
  std::memcpy(&h, host, sizeof(h));
  if (h.magic != kCkptMagic || h.version != 1) return fail(LBM_E_INVAL, "not a checkpoint");
  if (h.levels != g->levels || h.Q != g->Q || h.coll != g->coll || h.prec != g->prec || h.n_ranks != g->n_ranks ||
      h.rank != g->rank)
    return fail(LBM_E_INVAL, "checkpoint belongs to a different grid (levels/lattice/collision/precision/rank)");
  for (int L = 0; L < g->levels; ++L)
    if (h.nfluid[L] != g->host[L].nfluid || h.leaves[L] != g->host[L].leaves)
      return fail(LBM_E_INVAL, "checkpoint grid layout differs at level " + std::to_string(L));
  int64_t need = 0;
  lbm_checkpoint_size(g, &need);
  if (size < need) return fail(LBM_E_INVAL, "checkpoint truncated");
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  g->steps = h.steps;
  g->needs_prologue = h.needs_prologue != 0;
  const char* in = static_cast<const char*>(host);
  int64_t off = sizeof(h);
  for (int L = 0; L < g->levels; ++L) {
    const size_t b = pop_bytes(g, L);
    CUDA_TRY(cudaMemcpyAsync(g->dev[L].pop[cur_buf(g, L)], in + off, b, cudaMemcpyHostToDevice, g->stream));
    off += (int64_t)b;
  }
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  g->init_locked = h.steps > 0;
  return LBM_OK;
}

lbm_status lbm_profile_step(lbm_grid* g, int32_t n, double* level_ms, double* gather_ms, int64_t* launches_per_level) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (g->broken) return fail(LBM_E_STATE, "grid is in an error state");
  if (n < 0) return fail(LBM_E_INVAL, "n_coarse must be >= 0");
  for (int sd = 0; sd < 2; ++sd)
    if (g->n_ranks > 1 && g->has_nb[sd] && !g->connected[sd])
      return fail(LBM_E_STATE, "halo side " + std::to_string(sd) + " not connected");
  lbm_status s;
  if (g->needs_prologue && (s = run_prologue(g))) return s;
  std::vector<double> lms(g->levels, 0.0), gms(g->levels, 0.0);
  std::vector<int64_t> cnt(g->levels, 0);
  // One instrumented graph per parity of the step index: the coarse step's
  // launches in lbm_step's order, with a one-thread timestamp kernel node
  // (device global timer) before each level kernel's pre-kernels
  // (coalescence gather / volumetric averages / ablation kernels), between
  // them and the level kernel, and after it.  Replayed like lbm_step's graph,
  // so no host launch gaps are timed (CUDA event nodes in graphs cannot be
  // timed).  Eager launches instead under LBM_SCHED_NO_GRAPH.
  const size_t per = (size_t)1 << g->levels;  // > launches per coarse step
  void *dv = nullptr, *hv = nullptr;
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  if ((s = scratch_dev(g, 3 * per * sizeof(unsigned long long), &dv)) ||
      (s = scratch_host(g, 3 * per * sizeof(unsigned long long), &hv)))
    return s;
  unsigned long long* ts = static_cast<unsigned long long*>(dv);
  const unsigned long long* th = static_cast<const unsigned long long*>(hv);
  std::vector<std::pair<int, int64_t>> order[2];
  cudaGraphExec_t ge[2] = {nullptr, nullptr};
  auto cleanup = [&]() {
    for (int p = 0; p < 2; ++p)
      if (ge[p]) cudaGraphExecDestroy(ge[p]);
  };
  auto issue = [&](int par) {
    for (size_t j = 0; j < order[par].size(); ++j) {
      launch_stamp(ts, (int)(3 * j), g->stream);
      launch_F(g, order[par][j].first, order[par][j].second, 0, nullptr, ts + 3 * j + 1);
      launch_stamp(ts, (int)(3 * j + 2), g->stream);
    }
  };
  const bool eager = (g->sched & LBM_SCHED_NO_GRAPH) != 0;
  for (int i = 0; i < n; ++i) {
    const int par = (int)(g->steps & 1);
    step_order(g->levels, g->steps, order[par]);
    if (eager) {
      issue(par);
    } else {
      if (!ge[par]) {
        if (cudaStreamBeginCapture(g->stream, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
          cleanup();
          return fail(LBM_E_CUDA, "profile capture");
        }
        issue(par);
        cudaGraph_t graph = nullptr;
        cudaError_t le = cudaGetLastError();
        cudaError_t ce = cudaStreamEndCapture(g->stream, &graph);
        if (le != cudaSuccess || ce != cudaSuccess) {
          if (graph) cudaGraphDestroy(graph);
          cleanup();
          return fail(LBM_E_CUDA, std::string("profile capture: ") + cudaGetErrorString(le != cudaSuccess ? le : ce));
        }
        cudaError_t ie = cudaGraphInstantiate(&ge[par], graph, 0);
        cudaGraphDestroy(graph);
        if (ie != cudaSuccess) {
          cleanup();
          return fail(LBM_E_CUDA, std::string("profile instantiate: ") + cudaGetErrorString(ie));
        }
      }
      if (cudaGraphLaunch(ge[par], g->stream) != cudaSuccess) {
        cleanup();
        return fail(LBM_E_CUDA, "profile graph launch");
      }
    }
    cudaMemcpyAsync(hv, ts, 3 * order[par].size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream);
    cudaError_t se = cudaStreamSynchronize(g->stream);
    if (se != cudaSuccess) {
      cleanup();
      g->broken = true;
      return fail(LBM_E_CUDA, std::string("profile step: ") + cudaGetErrorString(se));
    }
    for (size_t j = 0; j < order[par].size(); ++j) {
      const int L = order[par][j].first;
      gms[L] += (double)(th[3 * j + 1] - th[3 * j]) * 1e-6;
      lms[L] += (double)(th[3 * j + 2] - th[3 * j + 1]) * 1e-6;
      cnt[L] += 1;
    }
    ++g->steps;
  }
  cleanup();
  for (int L = 0; L < g->levels; ++L) {
    if (level_ms) level_ms[L] = lms[L];
    if (gather_ms) gather_ms[L] = gms[L];
    if (launches_per_level) launches_per_level[L] = cnt[L];
  }
  g->init_locked = true;
  return LBM_OK;
}

lbm_status lbm_profile_levels(lbm_grid* g, int32_t n, double* ms_per_level, int64_t* launches_per_level) {
  std::vector<double> lms(g ? g->levels : 1), gms(g ? g->levels : 1);
  lbm_status s = lbm_profile_step(g, n, lms.data(), gms.data(), launches_per_level);
  if (s) return s;
  for (int L = 0; L < g->levels; ++L)
    if (ms_per_level) ms_per_level[L] = lms[L] + gms[L];
  return LBM_OK;
}

lbm_status lbm_synchronize(lbm_grid* g) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  return LBM_OK;
}

lbm_status lbm_macroscopic(lbm_grid* g, int32_t L, double* rho, double* u) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (L < 0 || L >= g->levels) return fail(LBM_E_INVAL, "level out of range");
  const HostLevel& H = g->host[L];
  // dense arrays over the owned slab of this rank (the whole level on one rank)
  const int64_t N = (H.owned_hi - H.owned_lo) * H.n[1] * H.n[2];
  const double nan = std::nan("");
  if (rho) std::fill(rho, rho + N, nan);
  if (u) std::fill(u, u + 3 * N, nan);
  const size_t chunk_cells = (size_t)kIoChunkBlocks * kCells;
  void *dv = nullptr, *hv = nullptr;
  lbm_status st;
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  if ((st = scratch_dev(g, chunk_cells * 4 * sizeof(double), &dv)) ||
      (st = scratch_host(g, chunk_cells * 4 * sizeof(double), &hv)))
    return st;
  const char* pop = static_cast<const char*>(g->dev[L].pop[cur_buf(g, L)]);
  for (int32_t b0 = 0; b0 < H.nlaunch; b0 += kIoChunkBlocks) {
    const int32_t nb = std::min(kIoChunkBlocks, H.nlaunch - b0);
    const size_t ncell = (size_t)nb * kCells;
    double* dr = static_cast<double*>(dv);
    launch_macroscopic(g->Q, g->prec, pop + (size_t)b0 * g->Q * kCells * g->tsize, g->dev[L].nbr + (size_t)b0 * kRec,
                       nb, dr, dr + ncell, nullptr, g->stream);
    CUDA_TRY(cudaGetLastError());
    CUDA_TRY(cudaMemcpyAsync(hv, dr, ncell * 4 * sizeof(double), cudaMemcpyDeviceToHost, g->stream));
    CUDA_TRY(cudaStreamSynchronize(g->stream));
    const double* r = static_cast<const double*>(hv);
    const double* v = r + ncell;
#pragma omp parallel for schedule(static)
    for (int32_t i = 0; i < nb; ++i) {
      const int32_t b = b0 + i;
      for (int l = 0; l < kCells; ++l) {
        if (H.types[(size_t)b * kCells + l] != kFluid) continue;
        const int64_t x = H.cell_x(b, l), y = H.cell_y(b, l), z = H.cell_z(b, l);
        if (x < H.owned_lo || x >= H.owned_hi) continue;
        const int64_t c = ((x - H.owned_lo) * H.n[1] + y) * H.n[2] + z;
        const size_t k = (size_t)i * kCells + l;
        if (rho) rho[c] = r[k];
        if (u) { u[3 * c] = v[3 * k]; u[3 * c + 1] = v[3 * k + 1]; u[3 * c + 2] = v[3 * k + 2]; }
      }
    }
  }
  return LBM_OK;
}

lbm_status lbm_probe(lbm_grid* g, int32_t L, int64_t n, const int64_t* xyz, double* rho, double* u) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (L < 0 || L >= g->levels) return fail(LBM_E_INVAL, "level out of range");
  if (n < 0 || (n > 0 && (!xyz || !rho || !u))) return fail(LBM_E_INVAL, "bad probe arguments");
  if (n == 0) return LBM_OK;
  const HostLevel& H = g->host[L];
  const int64_t xoff = (int64_t)g->x_lo << L;  // global -> local x (partitioned grids)
  const int64_t gnx = (int64_t)g->desc.nx << L;
  std::vector<int64_t> cell(n, -1);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    int64_t x = xyz[3 * i], y = xyz[3 * i + 1], z = xyz[3 * i + 2];
    if (x < 0 || x >= gnx || y < 0 || y >= H.n[1] || z < 0 || z >= H.n[2]) continue;
    x -= xoff;
    if (x < H.owned_lo || x >= H.owned_hi) continue;  // another rank's cell
    const int32_t b = H.block_at(x, y, z);
    if (b < 0 || b >= H.nlaunch) continue;
    const int l = H.local_at(x, y, z);
    if (H.types[(size_t)b * kCells + l] != kFluid) continue;
    cell[i] = (int64_t)b * kCells + l;
  }
  // scratch layout: cell indices, then rho[n], u[3n] (device); the same
  // through pinned host memory
  const size_t bytes = (size_t)n * (sizeof(int64_t) + 4 * sizeof(double));
  void *dv = nullptr, *hv = nullptr;
  lbm_status s;
  if ((s = scratch_dev(g, bytes, &dv)) || (s = scratch_host(g, bytes, &hv))) return s;
  // no wait for the queued steps here: every scratch user synchronises
  // before returning, so the pinned buffer is free and the upload, probe and
  // readback queue behind the step
  std::memcpy(hv, cell.data(), n * sizeof(int64_t));
  int64_t* dc = static_cast<int64_t*>(dv);
  double* dr = reinterpret_cast<double*>(dc + n);
  double* hr = reinterpret_cast<double*>(static_cast<int64_t*>(hv) + n);
  CUDA_TRY(cudaMemcpyAsync(dc, hv, n * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream));
  launch_probe(g->Q, g->prec, g->dev[L].pop[cur_buf(g, L)], dc, n, dr, dr + n, g->stream);
  CUDA_TRY(cudaGetLastError());
  CUDA_TRY(cudaMemcpyAsync(hr, dr, 4 * n * sizeof(double), cudaMemcpyDeviceToHost, g->stream));
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  std::memcpy(rho, hr, n * sizeof(double));
  std::memcpy(u, hr + n, 3 * n * sizeof(double));
  return LBM_OK;
}

lbm_status lbm_stats(lbm_grid* g, int64_t* leaves, double* mass) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  DeviceGuard dg_(g);
  if (leaves)
    for (int L = 0; L < g->levels; ++L) leaves[L] = g->host[L].leaves;
  if (!mass) return LBM_OK;
  // per-block mass partial sums of every level into one scratch buffer, one
  // D2H copy, one synchronisation
  size_t nb = 0;
  for (int L = 0; L < g->levels; ++L) nb += (size_t)std::max<int32_t>(g->host[L].nlaunch, 1);
  void *dv = nullptr, *hv = nullptr;
  lbm_status s;
  if ((s = scratch_dev(g, nb * sizeof(double), &dv)) || (s = scratch_host(g, nb * sizeof(double), &hv))) return s;
  double* bm = static_cast<double*>(dv);
  size_t off = 0;
  for (int L = 0; L < g->levels; ++L) {
    const HostLevel& H = g->host[L];
    launch_macroscopic(g->Q, g->prec, g->dev[L].pop[cur_buf(g, L)], g->dev[L].nbr, H.nlaunch, nullptr, nullptr,
                       bm + off, g->stream);
    off += (size_t)std::max<int32_t>(H.nlaunch, 1);
  }
  CUDA_TRY(cudaGetLastError());
  CUDA_TRY(cudaMemcpyAsync(hv, bm, nb * sizeof(double), cudaMemcpyDeviceToHost, g->stream));
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  const double* h = static_cast<const double*>(hv);
  double total = 0.0;
  off = 0;
  for (int L = 0; L < g->levels; ++L) {
    double sL = 0.0;
    for (int32_t b = 0; b < g->host[L].nlaunch; ++b) sL += h[off + b];
    off += (size_t)std::max<int32_t>(g->host[L].nlaunch, 1);
    total += sL * std::ldexp(1.0, -3 * L);
  }
  *mass = total;
  return LBM_OK;
}

lbm_status lbm_grid_get_info(const lbm_grid* g, lbm_grid_info* info) {
  g_err.clear();
  if (!g || !info) return fail(LBM_E_INVAL, "NULL argument");
  fill_info(g->host, g->Q, g->prec, g->n_ranks, info, g->sched, g->halo_spin, gather_spins(g));
  info->device_bytes = g->device_bytes;
  info->steps_done = g->steps;
  return LBM_OK;
}

lbm_status lbm_partition_cuts(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks, int32_t n_ranks,
                              int32_t* cuts) {
  g_err.clear();
  if (!cuts || n_ranks < 1) return fail(LBM_E_INVAL, "bad arguments");
  lbm_grid_desc dd = *d;
  dd.n_ranks = n_ranks;
  dd.rank = 0;
  lbm_status s = validate_desc(&dd, levels, masks);
  if (s) return s;
  std::vector<int32_t> c;
  partition_cuts(&dd, levels, masks, n_ranks, c);
  std::copy(c.begin(), c.end(), cuts);
  return LBM_OK;
}

lbm_status lbm_grid_slab(const lbm_grid* g, int32_t* x_begin, int32_t* x_end) {
  g_err.clear();
  if (!g) return fail(LBM_E_INVAL, "NULL grid");
  if (x_begin) *x_begin = g->cuts[g->rank];
  if (x_end) *x_end = g->cuts[g->rank + 1];
  return LBM_OK;
}

namespace {
struct HaloBlob {
  uint32_t magic, version;
  int32_t levels, Q, prec, side, rank, n_ranks;
  int32_t pid, device;
  char pci[32];  // PCI bus id of the exporter's GPU (same physical GPU -> halo_wait kernels)
  int64_t count[16];
  cudaIpcMemHandle_t pop[16][2];
  cudaIpcMemHandle_t flags;
};
constexpr uint32_t kBlobMagic = 0x484d424cu;  // "LBMH"

lbm_status invalidate_graphs(lbm_grid* g) {
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  for (int p = 0; p < 4; ++p)
    if (g->graph[p]) {
      cudaGraphExecDestroy(g->graph[p]);
      g->graph[p] = nullptr;
    }
  return LBM_OK;
}

lbm_status open_ipc(lbm_grid* g, const cudaIpcMemHandle_t& h, void** out) {
  std::string key(reinterpret_cast<const char*>(&h), sizeof(h));
  for (auto& e : g->ipc_open)
    if (e.first == key) { *out = e.second; return LBM_OK; }
  void* p = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) return fail(LBM_E_COMM, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
  g->ipc_open.push_back({key, p});
  *out = p;
  return LBM_OK;
}
}  // namespace

lbm_status lbm_halo_export(const lbm_grid* g, int32_t side, void* blob, int64_t capacity, int64_t* size) {
  g_err.clear();
  if (!g || side < 0 || side > 1) return fail(LBM_E_INVAL, "bad arguments");
  DeviceGuard dg_(g);
  if (g->n_ranks < 2 || !g->has_nb[side]) return fail(LBM_E_STATE, "no neighbour on this side");
  int64_t need = sizeof(HaloBlob);
  for (int L = 0; L < g->levels; ++L) need += (int64_t)g->host[L].halo[side].size() * 4;
  if (size) *size = need;
  if (!blob) return LBM_OK;
  if (capacity < need) return fail(LBM_E_INVAL, "blob capacity too small");
  HaloBlob h;
  std::memset(&h, 0, sizeof(h));
  h.magic = kBlobMagic;
  h.version = 1;
  h.levels = g->levels;
  h.Q = g->Q;
  h.prec = g->prec;
  h.side = side;
  h.rank = g->rank;
  h.n_ranks = g->n_ranks;
  h.pid = (int32_t)getpid();
  cudaGetDevice(&h.device);
  cudaDeviceGetPCIBusId(h.pci, (int)sizeof(h.pci), h.device);
  for (int L = 0; L < g->levels; ++L) {
    h.count[L] = (int64_t)g->host[L].halo[side].size();
    for (int b = 0; b < 2; ++b) CUDA_TRY(cudaIpcGetMemHandle(&h.pop[L][b], g->dev[L].pop[b]));
  }
  CUDA_TRY(cudaIpcGetMemHandle(&h.flags, g->flags));
  char* out = static_cast<char*>(blob);
  std::memcpy(out, &h, sizeof(h));
  int64_t off = sizeof(h);
  for (int L = 0; L < g->levels; ++L) {
    const auto& v = g->host[L].halo[side];
    std::memcpy(out + off, v.data(), v.size() * 4);
    off += (int64_t)v.size() * 4;
  }
  return LBM_OK;
}

static lbm_status check_counts(lbm_grid* g, int side, const int64_t* count) {
  for (int L = 0; L < g->levels; ++L)
    if (count[L] != (int64_t)g->host[L].send[side].size())
      return fail(LBM_E_COMM, "halo plan mismatch at level " + std::to_string(L) + ": neighbour expects " +
                                  std::to_string(count[L]) + " cells, this rank sends " +
                                  std::to_string(g->host[L].send[side].size()));
  return LBM_OK;
}

lbm_status lbm_halo_connect(lbm_grid* g, int32_t side, const void* blob, int64_t size) {
  g_err.clear();
  if (!g || !blob || side < 0 || side > 1) return fail(LBM_E_INVAL, "bad arguments");
  DeviceGuard dg_(g);
  if (g->n_ranks < 2 || !g->has_nb[side]) return fail(LBM_E_STATE, "no neighbour on this side");
  if (size < (int64_t)sizeof(HaloBlob)) return fail(LBM_E_INVAL, "blob too small");
  HaloBlob h;
  std::memcpy(&h, blob, sizeof(h));
  if (h.magic != kBlobMagic || h.version != 1) return fail(LBM_E_INVAL, "not a halo blob");
  if (h.side != 1 - side || h.levels != g->levels || h.Q != g->Q || h.prec != g->prec || h.n_ranks != g->n_ranks)
    return fail(LBM_E_COMM, "halo blob does not belong to this neighbour");
  if (h.pid == (int32_t)getpid()) return fail(LBM_E_INVAL, "same process: use lbm_halo_connect_local");
  lbm_status s = check_counts(g, side, h.count);
  if (s) return s;
  if ((s = invalidate_graphs(g))) return s;
  const char* in = static_cast<const char*>(blob);
  int64_t off = sizeof(h);
  for (int L = 0; L < g->levels; ++L) {
    DevLevel& D = g->dev[L];
    for (int b = 0; b < 2; ++b)
      if ((s = open_ipc(g, h.pop[L][b], &D.peer_pop[side][b]))) return s;
    std::vector<uint32_t> cells(h.count[L]);
    if (off + h.count[L] * 4 > size) return fail(LBM_E_INVAL, "blob truncated");
    std::memcpy(cells.data(), in + off, h.count[L] * 4);
    off += h.count[L] * 4;
    if ((s = dev_upload(g, &D.peer_cells[side], cells))) return s;
  }
  void* f = nullptr;
  if ((s = open_ipc(g, h.flags, &f))) return s;
  g->peer_flags[side] = static_cast<unsigned long long*>(f);
  {
    char mine[32] = {0};
    cudaDeviceGetPCIBusId(mine, (int)sizeof(mine), g->device);
    g->peer_other_gpu[side] = std::strncmp(mine, h.pci, sizeof(mine)) != 0;
  }
  // every local write to the buffers the peer stores into (zero-fill, init)
  // is complete before the caller's barrier lets the peer start stepping
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  CUDA_TRY(cudaDeviceSynchronize());
  g->connected[side] = true;
  update_halo_spin(g);
  return LBM_OK;
}

lbm_status lbm_halo_connect_local(lbm_grid* g, int32_t side, lbm_grid* peer) {
  g_err.clear();
  if (!g || !peer || side < 0 || side > 1) return fail(LBM_E_INVAL, "bad arguments");
  DeviceGuard dg_(g);
  if (g->n_ranks < 2 || !g->has_nb[side] || !peer->has_nb[1 - side]) return fail(LBM_E_STATE, "no neighbour");
  if (peer->levels != g->levels || peer->Q != g->Q || peer->prec != g->prec || peer->n_ranks != g->n_ranks)
    return fail(LBM_E_COMM, "peer grid does not match");
  int64_t count[16] = {0};
  for (int L = 0; L < g->levels; ++L) count[L] = (int64_t)peer->host[L].halo[1 - side].size();
  lbm_status s = check_counts(g, side, count);
  if (s) return s;
  if (peer->device != g->device) {
    // the level kernels store into the peer's buffers and bump its flags:
    // direct peer access over NVLink from this grid's device
    int ok = 0;
    CUDA_TRY(cudaDeviceCanAccessPeer(&ok, g->device, peer->device));
    if (!ok) return fail(LBM_E_COMM, "devices " + std::to_string(g->device) + " and " + std::to_string(peer->device) +
                                         " have no peer access");
    cudaError_t e = cudaDeviceEnablePeerAccess(peer->device, 0);
    if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
    else if (e != cudaSuccess) return fail(LBM_E_COMM, std::string("cudaDeviceEnablePeerAccess: ") + cudaGetErrorString(e));
  }
  if ((s = invalidate_graphs(g))) return s;
  for (int L = 0; L < g->levels; ++L) {
    DevLevel& D = g->dev[L];
    for (int b = 0; b < 2; ++b) D.peer_pop[side][b] = peer->dev[L].pop[b];
    if ((s = dev_upload(g, &D.peer_cells[side], peer->host[L].halo[1 - side]))) return s;
  }
  g->peer_flags[side] = peer->flags;
  CUDA_TRY(cudaStreamSynchronize(g->stream));
  CUDA_TRY(cudaStreamSynchronize(peer->stream));
  g->connected[side] = true;
  g->peer_other_gpu[side] = peer->device != g->device;
  update_halo_spin(g);
  return LBM_OK;
}

lbm_status lbm_halo_plan(const lbm_grid_desc* d, int32_t levels, const uint8_t* const* masks, int32_t side,
                         int32_t level, int64_t* send_xyz, int64_t* halo_xyz, int64_t capacity, int64_t* n_send,
                         int64_t* n_halo) {
  g_err.clear();
  if (side < 0 || side > 1 || level < 0 || level >= levels) return fail(LBM_E_INVAL, "bad side / level");
  lbm_status s = validate_desc(d, levels, masks);
  if (s) return s;
  if (d->n_ranks < 2) return fail(LBM_E_STATE, "single rank: no halo");
  std::vector<int32_t> cuts;
  partition_cuts(d, levels, masks, d->n_ranks, cuts);
  LocalSlab slab;
  make_local(d, levels, masks, cuts, slab);
  std::vector<HostLevel> host;
  if ((s = build_host(d, levels, masks, host, &slab))) return s;
  const HostLevel& H = host[level];
  if (n_send) *n_send = (int64_t)H.send[side].size();
  if (n_halo) *n_halo = (int64_t)H.halo[side].size();
  const int64_t gn = (int64_t)d->nx << level;
  auto put = [&](const std::vector<uint32_t>& v, int64_t* xyz) {
    if (!xyz) return;
    for (size_t i = 0; i < v.size() && (int64_t)i < capacity; ++i) {
      const uint32_t b = v[i] >> 9, l = v[i] & 511u;
      const int64_t x = H.cell_x((int32_t)b, (int)l);
      xyz[3 * i] = (((int64_t)slab.x_lo << level) + x + gn) % gn;
      xyz[3 * i + 1] = H.cell_y((int32_t)b, (int)l);
      xyz[3 * i + 2] = H.cell_z((int32_t)b, (int)l);
    }
  };
  put(H.send[side], send_xyz);
  put(H.halo[side], halo_xyz);
  return LBM_OK;
}

// the four halo-protocol counters (declared in lbmr.h as a debugging aid)
lbm_status lbm_debug_flags(lbm_grid* g, unsigned long long* out) {
  g_err.clear();
  if (!g || !out) return fail(LBM_E_INVAL, "NULL argument");
  if (!g->flags) return fail(LBM_E_STATE, "not a partitioned grid (no halo-protocol flags)");
  DeviceGuard dg_(g);
  cudaStream_t s;
  CUDA_TRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CUDA_TRY(cudaMemcpyAsync(out, g->flags, 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  cudaStreamDestroy(s);
  return LBM_OK;
}

void lbm_grid_destroy(lbm_grid* g) {
  if (!g) return;
  DeviceGuard dg_(g);
  if (g->stream) cudaStreamSynchronize(g->stream);
  for (int p = 0; p < 4; ++p)
    if (g->graph[p]) cudaGraphExecDestroy(g->graph[p]);
  for (auto& h : g->ipc_open) cudaIpcCloseMemHandle(h.second);
  if (g->scratch) cudaFree(g->scratch);
  if (g->hscratch) cudaFreeHost(g->hscratch);
  for (void* p : g->allocs) cudaFree(p);
  if (g->own_stream && g->stream) cudaStreamDestroy(g->stream);
  delete g;
}

}  // extern "C"
