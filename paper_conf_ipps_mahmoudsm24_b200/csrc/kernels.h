// kernels.h — launch interface of the sm_100a kernels (level_step.cu) used by
// the host runtime (capi.cpp).  No torch types; plain device pointers.
#pragma once
#include <cstdint>

#include <cuda_runtime.h>

namespace lbmr {

// Geometry of one level as the kernels see it (all pointers are device).
struct LevelView {
  int32_t n[3];             // cells per axis
  int32_t nb[3];            // blocks per axis
  const int32_t* blkmap;    // dense block map, -1 = no block
  const uint8_t* types;     // [nblocks][512] cell types (lattice.h codes)
};

struct BCEntry {
  int32_t kind;             // LBM_BC_NOSLIP / VELOCITY / OUTFLOW
  int32_t pad_;
  double u[3];              // wall / inlet velocity
};

// CTA size of the partitioned (halo-protocol) level kernels: a quarter of an
// 8^3 block; the host counts the protocol CTAs (nbctas) in these units.
constexpr int kHaloCtaThreads = 128;
constexpr int kHaloCtasPerBlock = 512 / kHaloCtaThreads;

// Parameters of one fused level-substep launch F_L^k: stream substep k of
// level L (pull, with BC, Explosion from L-1 and Coalescence from L+1), then
// collide substep k+1.
template <typename T>
struct StepParams {
  LevelView own, coarse, fine;
  const int32_t* nbr;           // [nfluid][kRec] block records (lattice.h)
  const int32_t* special_slot;  // [nfluid]
  const uint4* cellinfo;        // [nspecial][512] lattice.h kCellInfoWords layout
  const uint32_t* bmask;        // [nspecial][kBounceWords] per-warp bounce-mask unions
  const uint2* links;           // slow-link records (lattice.h kLink*)
  const uint32_t* coal;         // coalescence candidate lists
  const int32_t* origin;        // [nblocks][3] block coordinates
  const T* src;                 // C_L^k            [nfluid][Q][512]
  T* dst;                       // C_L^{k+1}
  const T* csrc;                // C_{L-1}^{ceil(k/2)}   (nullptr at L = 0)
  const T* fa;                  // C_{L+1}^{2k-1}        (nullptr at the finest level)
  const T* fb;                  // C_{L+1}^{2k}
  const BCEntry* bc;            // [256]
  T omega;                      // ω_L (Eq.9)
  int32_t periodic[3];
  const uint8_t* face_cls;      // [27] BC class of an out-of-domain source, by outside pattern
  int32_t nfluid;               // blocks launched (owned fluid blocks, cut-plane blocks first)
  // explosion ghosts of the destination buffer, refreshed from the coarse
  // post-collision state the NEXT kernel of this level reads (Eq.10)
  const uint32_t* ghost_fill;   // triples {ghost cell, parent cell, mask of the pulled directions}
  int32_t nghost;
  const T* gsrc;                // C_{L-1}^{ceil((k+1)/2)}
  // volumetric variant: when the next substep is the second
  // one of the parent's substep, the trailing CTAs evaluate these per-(ghost,
  // q) expressions (8 words each) instead of copying parents (nghost = 0)
  const uint32_t* vfill;
  int32_t nvfill;
  const T* vtemp;               // coarse averages of this level (kLinkTemp records)
  // ---- fusion-ablation schedules (lbm_set_schedule) --------
  // LBM_SCHED_ATOMIC_A (the paper's CA fusion): after colliding,
  // this level's CTAs add their post-collision values into the coarse
  // accumulators (the coalescence-ghost slots of C_{L-1}'s buffer `acc`) with
  // atomics, and the trailing CTAs reset this level's own accumulators in dst
  const uint32_t* zero_list;    // coalescence-ghost slots of dst to reset (nzero)
  int32_t nzero;
  const uint32_t* sc_qoff;      // [4 nfluid + 1] scatter items per 128-cell quarter block (CSR)
  const uint4* sc_items;        // {fine population index, coarse slot, |B|, 0}
  T* acc;                       // coarse buffer receiving the scatter (C_{L-1}^{ceil((k+1)/2)})
  int32_t sc_scaled;            // 1: add v / (2|B|) (division fused), 0: add v (separate O kernel)
  // Coalescence fused into this kernel (product schedule):
  // units of the Eq.11 gathers per 128-cell quarter-block CTA (grid_builder.h
  // cg_*), summed from fa / fb by warp shuffles into the CTA's shared column;
  // nullptr: the coalescence ghosts were filled by a gather kernel before
  const uint32_t* cg_qoff;      // [4 nfluid + 1]
  const uint32_t* cg_cand;      // [nunits][4]
  const uint32_t* cg_dest;      // [nunits]
  // 1: launched as the programmatic dependent (PDL) of the coalescence gather
  // that fills this kernel's coalescence ghosts: CTAs of blocks that pull
  // them (record word kRecCoalPull) wait for the gather at their start, all
  // others at their end, so the gather overlaps the level kernel
  int32_t pdl;
  // 1: launched as the programmatic dependent of the previous kernel of the
  // step (PDL chain): CTAs wait for it at their start, then trigger the next
  int32_t pdl_chain;
  // > 0: each block's first CTA prefetches (cp.async.bulk.prefetch.L2) the
  // populations of the block `prefetch` positions ahead in storage order
  int32_t prefetch;
  // ---- x-slab partition (multi-GPU); unused when nbctas == 0 -------------
  int32_t nbctas;               // CTAs taking part in the halo protocol (cut-plane blocks, >= 1)
  int32_t nboundary;            // cut-plane blocks (stored and launched first)
  int32_t has_nb[2];            // neighbour on the -x / +x side
  int32_t halo_spin;            // 1: protocol CTAs wait in-kernel (neighbours on other GPUs), 0: halo_wait_kernel
  unsigned long long* flags;    // this rank: [0],[1] bumped by the -x/+x neighbour, [2] kernels done, [3] CTA count
  unsigned long long* peer_flag[2];  // neighbour's flag slot this rank bumps
  T* peer_dst[2];               // neighbour's C_L^{k+1} buffer
  const uint32_t* peer_cells[2];     // neighbour's halo cell index for each entry of my send list
  const int32_t* bpeer;         // [nboundary][2][512] send-list index of a cut-plane cell, or -1
};

// Coalescence gather (Eq.11) into the coarse ghosts of `dst` (= C_L^k's
// buffer, read next by F_L^k): for entry i, dst[fill[i]] = (sum_B fa + sum_B fb)
// / (2|B|) over the filled candidate slots of entry i (grid_builder.h
// coal_cand: n_main entries with kCoalSlots slots, then n_ovf entries with
// kCoalSlotsMax slots, structure-of-arrays).
// mode (kCoal*): kCoalFromDst starts each sum from dst[fill[i]] instead of 0,
// kCoalDivide divides the sum by 2|B|; fa / fb may be NULL (that source is
// skipped).  The product schedule's gather is (fa, fb, kCoalDivide); the
// ablation schedules split it into Accumulate (fa or fb only, no division)
// and Coalescence O (no source, kCoalFromDst | kCoalDivide) kernels.
enum { kCoalFromDst = 1, kCoalDivide = 2 };
// spin_flags (partitioned grid whose neighbours are on other GPUs): every CTA
// first waits in-kernel for the neighbours' previous kernels (halo protocol).
// pdl_chain: launched as the programmatic dependent of the previous level
// kernel (it waits for it at entry).
void launch_coalesce(int Q, int precision, const void* fa, const void* fb, void* dst, const uint32_t* fill,
                     const uint32_t* cand, int64_t n_main, int64_t n_ovf, int mode, cudaStream_t s,
                     const unsigned long long* spin_flags = nullptr, int nb0 = 0, int nb1 = 0,
                     int pdl_chain = 0);

// The same gather, warp-cooperative: 4 lanes per 4-slot unit (grid_builder.h
// coal_wcand / coal_wdst; units [pair, n) form |B| > 4 pairs), the values
// added by warp shuffles in the order of launch_coalesce (bitwise equal).
void launch_coalesce_warp(int precision, const void* fa, const void* fb, void* dst, const uint32_t* cand,
                          const uint32_t* udst, int64_t n_units, int64_t pair, int mode, cudaStream_t s,
                          const unsigned long long* spin_flags = nullptr, int nb0 = 0, int nb1 = 0,
                          int pdl_chain = 0);

// rho / u (double) of n cells given by population cell index block*512+local
// (-1 -> NaN), read from the post-collision buffer `pop`.
void launch_probe(int Q, int precision, const void* pop, const int64_t* cell, int64_t n, double* rho, double* u,
                  cudaStream_t s);

// Volumetric variant: coarse averages of level L before F_L^k.
// ent: [n][36] {slot, 0, 0, 0, 8 expressions}; A = C_L^k, B = C_{L+1}^{2k-1},
// C = C_{L+1}^{2k}; tmp[n] receives the means; then the slots are written.
void launch_vavg(int Q, int precision, const uint32_t* ent, int32_t n, void* A, const void* B, const void* C,
                 const BCEntry* bc, const uint8_t* face_cls, void* tmp, cudaStream_t s);

// One-thread kernel: wait until both neighbours (has_nb) have completed the
// cut-plane part of every kernel this rank has completed.
void launch_halo_wait(const unsigned long long* flags, int nb0, int nb1, cudaStream_t s);

// lbm_set_bc's device update: the BC entry of one class and the 27 face
// classes travel as kernel arguments (copied at launch), so the host call
// neither waits for the stream nor keeps a host buffer alive.
struct FaceTable {
  uint8_t cls[28];
};
void launch_bc_update(BCEntry* bc, int cls, BCEntry e, uint8_t* face_cls, FaceTable ft, cudaStream_t s);

// One-thread kernel writing the device global timer (ns) into out[idx].
void launch_stamp(unsigned long long* out, int idx, cudaStream_t s);

// Force-load every kernel (see level_step.cu).
void preload_kernels();

// kind: 0 = fused stream+collide F_L^k, 1 = collide only (prologue C_L^1,
// src -> dst), 3 = stream only S_L^k (unfused schedule, with the explosion
// ghost refresh), 4 = collide dst in place (unfused schedule), 5 = Explosion
// only: refresh the explosion ghosts of dst from gsrc (ablation E kernel)
void launch_level_step(int Q, int collision, int precision, int kind, const void* params, cudaStream_t s);

// g = f^eq(rho,u) - w on the fluid cells of `nfluid` blocks; rho/u compact
// device arrays [nfluid*512] and [nfluid*512*3] (double).
void launch_init_eq(int Q, int precision, void* pop, const uint8_t* types, int32_t nfluid,
                    const double* rho, const double* u, cudaStream_t s);

// rho/u (double, compact, NaN on cells that are not owned fluid leaves) of the
// post-collision buffer `pop`; optional per-block mass partial sums
// block_mass[nblk].  rec = block records (lattice.h kRec*).
void launch_macroscopic(int Q, int precision, const void* pop, const int32_t* rec, int32_t nblk,
                        double* rho, double* u, double* block_mass, cudaStream_t s);

}  // namespace lbmr
