/*
 * lbmr.h — C ABI of the B200-native multi-level grid-refinement LBM library
 * (liblbmr.so).  One coarse time step of nonuniform grid refinement LBM in the
 * volume-based style of Rohde et al. [25] as optimised by Mahmoud,
 * Salehipour and Meneghin (IPDPS 2024).  Citations "P:Lnnn" are lines of
 * /root/reference/PAPER.md with the section / equation they fall in.
 *
 * Conventions shared by every call
 * --------------------------------
 *  - Levels L = 0 (coarsest) .. levels-1.  Level L has (nx<<L, ny<<L, nz<<L)
 *    cells; refinement ratio 2 (§II-A), acoustic scaling: level L runs
 *    2^L substeps per coarse step (§III).
 *  - Host arrays are C-order, z fastest: cell (x,y,z) of level L has linear
 *    index (x*(ny<<L) + y)*(nz<<L) + z.  Velocity arrays are interleaved
 *    [cell][3].  All host arrays are owned by the caller; the library copies
 *    what it needs during the call and keeps no pointer.
 *  - Cell codes in masks (uint8): 0 = not a leaf at this level (REFINED if
 *    its children are covered, ABSENT if a coarser leaf covers it), 1 = fluid
 *    leaf, 2..254 = boundary-condition leaf of that class id, 255 reserved.
 *  - Device memory: the library allocates and owns all device memory
 *    (populations, 2 buffers per level, and the block tables); freed by
 *    lbm_grid_destroy.  Work is enqueued on the grid's stream.
 *  - Errors: no exception crosses the ABI.  Every call returns an
 *    lbm_status; on a non-OK status lbm_last_error() holds a thread-local
 *    text.  A grid whose lbm_step failed is in LBM_E_STATE until destroyed.
 *    CUDA errors of asynchronous work surface at the next synchronising call
 *    (lbm_macroscopic, lbm_stats, lbm_synchronize).
 */
#ifndef LBMR_H
#define LBMR_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  LBM_OK = 0,
  LBM_E_INVAL = 1,       /* bad argument (NULL pointer, bad enum, bad dims)          */
  LBM_E_TILING = 2,      /* masks do not tile the domain exactly once       */
  LBM_E_UNBALANCED = 3,  /* two 26-adjacent leaves differ by > 1 level */
  LBM_E_OOM = 4,         /* device or host allocation failed                          */
  LBM_E_CUDA = 5,        /* CUDA runtime error (text in lbm_last_error)               */
  LBM_E_COMM = 6,        /* multi-GPU exchange error                                   */
  LBM_E_STATE = 7,       /* call not valid in the grid's current state                 */
  LBM_E_UNSUPPORTED = 8  /* valid request this build does not implement (KBC+D3Q19)   */
} lbm_status;

typedef enum { LBM_D3Q19 = 19, LBM_D3Q27 = 27 } lbm_lattice;       /* P:L37 §II          */
typedef enum { LBM_BGK = 0, LBM_KBC = 1 } lbm_collision;           /* Eq.3; KBC [18] (D3Q27 only) */
typedef enum { LBM_FP32 = 0, LBM_FP64 = 1 } lbm_precision;         /* fp32 stores shifted populations f - w */
typedef enum {
  LBM_BC_NOSLIP = 0,    /* halfway bounce-back [27]                          */
  LBM_BC_VELOCITY = 1,  /* moving wall / velocity inlet: bounce-back + 6 w_i rho_w e_i.u_w,
                           rho_w = 1 (P:L264 lid, P:L280 inlet)                                */
  LBM_BC_OUTFLOW = 2    /* missing f_i := w_i                                         */
} lbm_bc_kind;

typedef struct {
  int32_t nx, ny, nz;       /* level-0 cells per axis (>= 1)                                 */
  int32_t periodic[3];      /* 1 = periodic axis; non-periodic faces use face_bc             */
  uint8_t face_bc[6];       /* BC class (2..254) of sources outside the -x,+x,-y,+y,-z,+z
                               faces; at edges/corners VELOCITY > NOSLIP > OUTFLOW           */
  uint8_t pad_[2];
  int32_t lattice;          /* lbm_lattice                                                   */
  int32_t collision;        /* lbm_collision                                                 */
  int32_t precision;        /* lbm_precision                                                 */
  double omega0;            /* level-0 relaxation Δt/τ; ω_L by Eq.9                 */
  int32_t n_ranks, rank;    /* x-slab partition; (1, 0) = whole domain on this device        */
  void* stream;             /* cudaStream_t to enqueue on; NULL = library-owned stream      */
  int32_t variant;          /* LBM_VARIANT_PAPER (0): the paper's method as read in DESIGN.md
                               §3 (default).  LBM_VARIANT_VOLUMETRIC (1): fine-ghost advection,
                               mass-exact on interface edges/corners (single
                               rank; LBM_E_UNSUPPORTED where a wall touches the coarse side of
                               an interface in a way the traces cannot express)              */
} lbm_grid_desc;
enum { LBM_VARIANT_PAPER = 0, LBM_VARIANT_VOLUMETRIC = 1 };

typedef struct lbm_grid lbm_grid;

typedef struct {
  int32_t levels;
  int32_t Q;
  int32_t precision;
  int32_t kernels_per_step;          /* 2^levels - 1 fused level-step launches (pipelined Alg.1) */
  int64_t leaves[16];                /* fluid leaves per level                                   */
  int64_t blocks[16];                /* 8^3 blocks holding >= 1 fluid leaf                        */
  int64_t special_blocks[16];        /* blocks with a non-same-level or BC link                   */
  int64_t special_cells[16];         /* fluid leaves with such a link                             */
  int64_t total_blocks[16];          /* all stored blocks incl. refined/BC-only                   */
  int64_t device_bytes;              /* device memory held by the grid                            */
  int64_t steps_done;                /* coarse steps since the last init                          */
  int64_t launches_per_step;         /* every kernel of one coarse step under the current schedule:
                                        the level steps (the product gathers coalescence inside
                                        them), plus the separate gather / split kernels and halo
                                        waits other schedules add                                   */
  int32_t block_offset[16][3];       /* per level and axis: level cell c lies in 8^3 block
                                        (c + off) >> 3 (builder-chosen alignment)     */
  int64_t coal_links[16];            /* per level: coalescence links with B != {} (Eq.11 gathers
                                        per F_L^k)                                                  */
  int64_t coal_wide[16];             /* of those, links with |B| > 4 (concave interface edges)      */
} lbm_grid_info;

/* Build the block-sparse multi-level grid (§V) from per-level masks.
 * masks[L] points to (nx<<L)*(ny<<L)*(nz<<L) codes (see conventions).  Validates
 * exact tiling (LBM_E_TILING) and strong 2:1 balance over the 26-neighbourhood
 * (LBM_E_UNBALANCED), the first offending level/cell going to lbm_last_error.
 * Allocates device memory; populations start at rest equilibrium (rho=1, u=0).
 * levels in [1, 16]; KBC requires D3Q27 (LBM_E_UNSUPPORTED otherwise). */
lbm_status lbm_grid_create(const lbm_grid_desc* desc, int32_t levels, const uint8_t* const* masks,
                           lbm_grid** out);

/* Define boundary class `bc_class` (2..254): kind and wall velocity u_wall[3]
 * (lattice units of the level the link lives on; NULL = 0).  Takes effect at
 * the next lbm_step.  Undefined classes used by masks/face_bc act as NOSLIP.
 * Asynchronous: the entry and the recomputed edge/corner face classes are
 * enqueued on the grid's stream as kernel arguments (no host wait, no host
 * buffer kept), so they apply to steps launched after this call only. */
lbm_status lbm_set_bc(lbm_grid* g, int32_t bc_class, int32_t kind, const double* u_wall);

/* f = f^eq(rho, u) (Eq.5) on the fluid leaves of `level`.  rho: dense
 * level array or NULL (= 1); u: dense interleaved [cell][3] or NULL (= 0).
 * Resets the step counter; the next lbm_step starts from this post-streaming
 * state. */
lbm_status lbm_init_equilibrium(lbm_grid* g, int32_t level, const double* rho, const double* u);

/* f = f^eq(rho0, u0) on every fluid leaf of every level (u0 NULL = 0). */
lbm_status lbm_init_uniform(lbm_grid* g, double rho0, const double* u0);

/* Advance n_coarse coarse time steps (Algorithm 1): the fused
 * per-level kernels {pull streaming + BC, Explosion Eq.10, Coalescence Eq.11
 * (gather form of Accumulate), Collision Eq.3 / KBC} in the pipelined
 * order, replayed as a CUDA graph.  Asynchronous on the grid's stream. */
lbm_status lbm_step(lbm_grid* g, int32_t n_coarse);

/* rho (Eq.6) and u (Eq.7) of level `level` into dense host arrays (rho: cells,
 * u: cells*3 interleaved; either may be NULL).  Cells that are not fluid
 * leaves get NaN.  Synchronises the grid's stream. */
lbm_status lbm_macroscopic(lbm_grid* g, int32_t level, double* rho, double* u);

/* Probes (also the sampled full-size parity checks):
 * rho (Eq.6) and u (Eq.7) at n cells of level `level` given as GLOBAL
 * level-L integer coordinates xyz[3n] (x, y, z).  rho[n] and u[3n] are
 * caller-owned host arrays.  Cells that are outside the domain, not fluid
 * leaves of this level, or owned by another rank of a partition get NaN.
 * Synchronises the grid's stream. */
lbm_status lbm_probe(lbm_grid* g, int32_t level, int64_t n, const int64_t* xyz, double* rho, double* u);

/* Fluid leaves per level (leaves_per_level[levels], may be NULL) and total
 * mass sum_L sum_leaves rho * 8^-L in coarse-cell volumes (may be NULL).
 * Synchronises. */
lbm_status lbm_stats(lbm_grid* g, int64_t* leaves_per_level, double* total_mass);

/* Grid description and sizes (no device work).  launches_per_step counts every
 * kernel one coarse step launches (level kernels, coalescence gathers, the
 * halo waits of a partitioned grid); device_bytes equals what
 * lbm_grid_analyze predicts for the same desc/masks (scratch buffers of the
 * diagnostics calls, allocated on demand, are not included). */
lbm_status lbm_grid_get_info(const lbm_grid* g, lbm_grid_info* info);

/* Instrumented run for measurement: advances n_coarse steps replaying, per
 * parity of the step index, a CUDA graph of the same launches as lbm_step's
 * with a one-thread timestamp kernel (device global timer) before each level
 * kernel's pre-kernels (coalescence gather / volumetric averages / ablation
 * kernels), between them and the level kernel, and after it (eager launches
 * instead under LBM_SCHED_NO_GRAPH).  level_ms[L]: summed
 * device time of level L's kernels F_L^k; gather_ms[L]: of the pre-kernels
 * feeding them; launches_per_level[L]: number of F_L^k (any may be NULL).
 * Synchronises after every step. */
lbm_status lbm_profile_step(lbm_grid* g, int32_t n_coarse, double* level_ms, double* gather_ms,
                            int64_t* launches_per_level);

/* lbm_profile_step with ms_per_level[L] = level_ms[L] + gather_ms[L]. */
lbm_status lbm_profile_levels(lbm_grid* g, int32_t n_coarse, double* ms_per_level,
                              int64_t* launches_per_level);

/* Kernel schedule of lbm_step / lbm_profile_* (bit flags; default 0).  The
 * steps of one level-substep are C (collision), A (Accumulate: fine
 * post-collision values into the coarse-side ghost layer), S (streaming),
 * E (Explosion) and O (Coalescence: the coarse level reads and averages the
 * accumulated values), §IV and Fig. 4.
 *  LBM_SCHED_FUSED     (0) one fused kernel F_L^k per level-substep (S + E +
 *                      O + BC + C), 2Q values moved per leaf, and one small
 *                      gather kernel before it doing A + A + O from the two
 *                      retained fine buffers (deterministic, one thread per
 *                      link; F_L^k its programmatic dependent) — the product.
 *                      (LBMR_GATHER_WARP=1 in the environment at grid creation
 *                      selects a warp-cooperative form of the same gather:
 *                      bitwise equal, measured slower.)
 *  LBM_SCHED_UNFUSED   (1) C and S separate: a stream-only kernel S_L^k then
 *                      an in-place collision C_L^{k+1} (4Q values per leaf).
 *  LBM_SCHED_NO_GRAPH  (2) launch the kernels one by one instead of replaying
 *                      the captured CUDA graph (launch-overhead ablation).
 *  LBM_SCHED_SPLIT_E   (4) E separate: an Explosion kernel refreshes the
 *                      level's explosion ghosts before its S / F kernel.
 *  LBM_SCHED_SPLIT_A   (8) A separate, as a gather initiated from the coarse
 *                      level after every fine Collision (raw sums into the
 *                      coarse ghost slots; the paper's modified baseline).
 *  LBM_SCHED_ATOMIC_A  (16) A fused into the fine Collision as a scatter
 *                      atomic write (CA, Fig. 4c); the coarse
 *                      kernel resets the ghost layer.  Summation order is not
 *                      deterministic (results differ from the others by
 *                      rounding only).
 *  LBM_SCHED_SPLIT_O   (32) O's division by 2|B| as its own kernel before
 *                      the coarse S / F (otherwise fused into the last
 *                      Accumulate, or pre-scaled atomic terms).
 *  LBM_SCHED_CTA_GATHER (64) A + A + O inside F_L^k instead of the gather
 *                      kernel: each CTA first gathers its own cells'
 *                      coalescence links (warp shuffles, into its shared
 *                      staging column); ignored with UNFUSED, SPLIT_A,
 *                      ATOMIC_A or SPLIT_O (which need the ghost slots).
 * The paper's configurations: Fig. 4b modified baseline = UNFUSED | SPLIT_E |
 * SPLIT_A | SPLIT_O; 4c = UNFUSED | SPLIT_E | ATOMIC_A | SPLIT_O; 4d (SE
 * fused) = UNFUSED | SPLIT_A | SPLIT_O; 4e (CA, SE, SO fused) = UNFUSED |
 * ATOMIC_A; 4f (CASE and SO fused) = ATOMIC_A.  All non-atomic schedules are
 * bitwise identical to LBM_SCHED_FUSED.  Every bit except NO_GRAPH is single
 * rank, paper variant only (LBM_E_UNSUPPORTED).  Switching at a coarse-step
 * boundary is allowed (pending accumulations are rebuilt).  Takes effect at
 * the next lbm_step; synchronises the grid's stream. */
enum {
  LBM_SCHED_FUSED = 0,
  LBM_SCHED_UNFUSED = 1,
  LBM_SCHED_NO_GRAPH = 2,
  LBM_SCHED_SPLIT_E = 4,
  LBM_SCHED_SPLIT_A = 8,
  LBM_SCHED_ATOMIC_A = 16,
  LBM_SCHED_SPLIT_O = 32,
  LBM_SCHED_CTA_GATHER = 64
};
lbm_status lbm_set_schedule(lbm_grid* g, int32_t mode);

/* Checkpoint / resume.  The state at a coarse-step
 * boundary is, per level, the current population buffer (post-collision
 * C_L^{k+1} with its explosion/coalescence ghosts, or the initial
 * post-streaming state before the first step) plus the step counter.
 *  lbm_checkpoint_size:  bytes a checkpoint of this grid takes (header +
 *                        sum_L blocks_L * Q * 512 * sizeof(precision)).
 *  lbm_checkpoint_save:  synchronises, copies the state into the caller's
 *                        host buffer `host` of `capacity` bytes
 *                        (LBM_E_INVAL if too small).
 *  lbm_checkpoint_load:  restores a checkpoint into a grid created from the
 *                        SAME desc/masks (same rank of the same partition);
 *                        LBM_E_INVAL if it belongs to another layout.  The
 *                        continued run is bitwise identical to an
 *                        uninterrupted one.  The caller owns `host`. */
lbm_status lbm_checkpoint_size(const lbm_grid* g, int64_t* bytes);
lbm_status lbm_checkpoint_save(lbm_grid* g, void* host, int64_t capacity);
lbm_status lbm_checkpoint_load(lbm_grid* g, const void* host, int64_t size);

/* Block until all work enqueued on the grid's stream is done. */
lbm_status lbm_synchronize(lbm_grid* g);

/* Destroy the grid and free its device memory; NULL is a no-op.  Waits for the
 * grid's own stream only: on a partitioned grid the neighbours' kernels store
 * into this grid's buffers, so every rank must synchronise its grid and pass a
 * barrier before any rank destroys its grid (PartitionedGrid.close does this
 * for grids of one process). */
void lbm_grid_destroy(lbm_grid* g);

/* Thread-local text of the last non-OK status ("" if none). */
const char* lbm_last_error(void);

/* Library version string. */
const char* lbm_version(void);

/* ---- host-only helpers (no CUDA device needed) -------------------------- */

/* Validate masks and build the block tables on the host only, filling the
 * counts of `info` (levels, Q, leaves, blocks, special blocks/cells,
 * kernels_per_step); device_bytes is the population + table footprint
 * lbm_grid_create allocates (the same allocation list).  Same validation and error codes as lbm_grid_create. */
lbm_status lbm_grid_analyze(const lbm_grid_desc* desc, int32_t levels, const uint8_t* const* masks,
                            lbm_grid_info* info);

/* The pipelined launch order of coarse step n (0-based) for `levels` levels:
 * writes pairs (level, k) of F_L^k (stream substep k of level L, collide
 * substep k+1) into order[2*i], order[2*i+1] for i < 2^levels - 1.  Returns
 * the number of launches, or -1 if levels is out of [1, 16] / order is NULL. */
int32_t lbm_schedule(int32_t levels, int64_t n, int64_t* order, int32_t capacity);

/* The library's lattice: e[Q][3] velocities and w[Q] weights in the order the
 * kernels use (rest first, then opposite pairs).  Returns Q, or -1. */
int32_t lbm_lattice_table(int32_t Q, int32_t* e, double* w);

/* Relaxation rate of level L from omega0, Eq.(9) P:L100. */
double lbm_omega_level(double omega0, int32_t level);

/* ---- x-slab partition (multi-GPU), DESIGN.md §9 ---------------------------
 * A grid created with desc->n_ranks = P > 1 holds rank desc->rank's slab of
 * level-0 x cells [cuts[rank], cuts[rank+1]) (cuts from lbm_partition_cuts,
 * identical on every rank since they depend only on the masks) plus one
 * level-0 cell of halo on each side that has a neighbour (x periodic: a ring).
 * Every rank passes the SAME global masks.  Dense arrays of
 * lbm_init_equilibrium / lbm_macroscopic then cover the owned slab only:
 * shape ((cuts[rank+1]-cuts[rank])<<L, ny<<L, nz<<L).  Before the first
 * lbm_step every side with a neighbour must be connected (lbm_halo_connect
 * with the neighbour's lbm_halo_export blob, or lbm_halo_connect_local for a
 * grid of the same process); all ranks must then issue the same sequence of
 * lbm_step / lbm_profile_levels calls.  Side 0 = -x, side 1 = +x. */

/* Balanced cuts (n_ranks + 1 entries) at level-0 cell boundaries: the work of
 * column x is sum_L 2^L (fluid leaves of level L inside it).  Host only. */
lbm_status lbm_partition_cuts(const lbm_grid_desc* desc, int32_t levels, const uint8_t* const* masks,
                              int32_t n_ranks, int32_t* cuts);

/* Owned level-0 x range [x_begin, x_end) of the grid (global coordinates). */
lbm_status lbm_grid_slab(const lbm_grid* g, int32_t* x_begin, int32_t* x_end);

/* Serialise what the neighbour on `side` needs to write into this grid: the
 * halo cell lists per level and CUDA IPC handles of the population buffers
 * and the protocol flags.  blob = NULL returns the size only. */
lbm_status lbm_halo_export(const lbm_grid* g, int32_t side, void* blob, int64_t capacity, int64_t* size);

/* Connect `side` to the neighbour whose lbm_halo_export(other side) blob is
 * given (another process; the buffers are opened with CUDA IPC). */
lbm_status lbm_halo_connect(lbm_grid* g, int32_t side, const void* blob, int64_t size);

/* Connect `side` to a neighbour grid of this process (same device or a
 * peer-accessible one). */
lbm_status lbm_halo_connect_local(lbm_grid* g, int32_t side, lbm_grid* peer);

/* Debugging aid: the four halo-protocol counters of a partitioned grid
 * (out[4]: [0]/[1] bumped by the -x/+x neighbour per finished kernel, [2]
 * kernels finished by this rank, [3] protocol CTAs of the running kernel),
 * read on a separate stream without waiting for the grid's stream.
 * LBM_E_STATE on a single-rank grid. */
lbm_status lbm_debug_flags(lbm_grid* g, unsigned long long* out);

/* Host-only plan of one side/level of rank desc->rank: global coordinates
 * (x, y, z) of the cells it sends (its first owned layer at the cut) and of
 * its halo cells (received), in the order both sides use.  xyz arrays hold
 * 3 * capacity int64 each (may be NULL to query the counts). */
lbm_status lbm_halo_plan(const lbm_grid_desc* desc, int32_t levels, const uint8_t* const* masks, int32_t side,
                         int32_t level, int64_t* send_xyz, int64_t* halo_xyz, int64_t capacity, int64_t* n_send,
                         int64_t* n_halo);

#ifdef __cplusplus
}
#endif

#endif /* LBMR_H */
