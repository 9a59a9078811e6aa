// grid_builder.h — host construction of the block-sparse multi-level grid
// (§V-A/B): masks -> validated leaf tiling -> per level 8^3 blocks
// in Morton order, dense block map, per-block cell types, neighbour-block
// table, per-cell slow-link masks.  Pure host C++ (OpenMP), no CUDA.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace lbmr {

struct HostLevel {
  int64_t n[3] = {0, 0, 0};      // cells per axis
  int32_t nb[3] = {0, 0, 0};     // blocks per axis (ceil((n + off) / 8))
  // block-grid offset per axis: level cell x lies in block (x + off) >> 3 at
  // local position (x + off) & 7.  Chosen by the builder to put the level's
  // fluid-region faces on block faces (whole 32-byte rows);
  // always 0 on periodic axes.
  int32_t off[3] = {0, 0, 0};
  int32_t nblocks = 0;           // stored blocks (fluid first)
  int32_t nfluid = 0;            // blocks holding >= 1 fluid leaf
  int32_t nspecial = 0;          // fluid blocks with a non-trivial cell
  int64_t leaves = 0;            // fluid leaves
  int64_t special_cells = 0;     // fluid leaves with >= 1 slow link
  std::vector<int32_t> blkmap;   // [nb0*nb1*nb2] block id or -1; index (bx*nb1+by)*nb2+bz
  std::vector<int32_t> origin;   // [nblocks*3] block coordinates
  std::vector<uint8_t> types;    // [nblocks*512] cell type (lattice.h codes), local = x+8y+64z
  std::vector<int32_t> nbr;      // [nfluid*kRec] block records (lattice.h: neighbours, slot, origin)
  std::vector<int32_t> special_slot;  // [nfluid] index into cellinfo or -1 (plain block)
  std::vector<uint32_t> cellinfo;     // [nspecial*512][kCellInfoWords] (lattice.h)
  std::vector<uint32_t> bmask;        // [nspecial][kBounceWords] per-warp union of the bounce masks
  std::vector<uint32_t> links;        // [nlinks][2] slow-link records (lattice.h kLink*)
  std::vector<uint32_t> coal;         // coalescence candidate population indices
  int64_t nlinks = 0;
  // partition (empty / zero on a single rank)
  int32_t nlaunch = 0;                // blocks with owned fluid leaves (launched), boundary ones first
  int32_t nboundary = 0;              // launched blocks holding an owned cell of a cut plane
  int64_t owned_lo = 0, owned_hi = 0; // owned x range at this level (local coordinates)
  std::vector<uint32_t> send[2];      // owned fluid cells of the first layer at each cut, (y,z) order
  std::vector<uint32_t> halo[2];      // halo fluid cells just outside each cut, (y,z) order
  std::vector<int32_t> bpeer;         // [nboundary][2][512] index into send[side] or -1
  // explosion ghosts (ABSENT cells pulled by fluid leaves, parent a fluid
  // leaf at L-1): stored, refreshed by the level's previous kernel
  std::vector<uint8_t> ghost;         // [nblocks*512] host only: 1 explosion ghost, 2 coalescence ghost
  std::vector<uint32_t> ghost_fill;   // triples {ghost cell at L, parent cell at L-1 (block*512+local), pulled-q mask}
  std::vector<uint32_t> coal_fill;    // [n] dest population index (ghost, q), sorted by (q, dest) per segment
  std::vector<uint32_t> coal_cand;    // SoA fine candidate population indices (level L+1), ~0u = empty:
                                      // [kCoalSlots][coal_n[0]] then [kCoalSlotsMax][coal_n[1]]
  int64_t coal_n[2] = {0, 0};         // entries with |B| <= kCoalSlots, and the others
  // the same gather list for the warp-cooperative gather kernel: 4-slot units
  // (array of structures, one 16-byte unit per 4 lanes), the entries with
  // |B| <= 4 first, then the others as two units each starting at an even
  // unit (one warp holds both); destination population index per unit (~0u:
  // second unit of a pair, or padding)
  std::vector<uint32_t> coal_wcand;   // [nunits][4]
  std::vector<uint32_t> coal_wdst;    // [nunits]
  int64_t coal_wpair = 0;             // first unit of the pair segment
  // Coalescence fused into the coarse level kernel (product schedule,
  // DESIGN.md §6): per 128-cell quarter block of a launched block, the Eq.11
  // gathers its own fluid leaves need, as units of 4 candidate slots (an
  // entry with |B| > 4 takes two consecutive units, the first never the last
  // of an 8-unit warp group, so one warp holds both)
  std::vector<uint32_t> cg_qoff;      // [4 nlaunch + 1] CSR offsets into the units
  std::vector<uint32_t> cg_cand;      // [nunits][4] fine candidate population indices (level L+1), ~0u = empty
  std::vector<uint32_t> cg_dest;      // [nunits] quarter-local cell | q << 7 | kind << 12 (lattice.h kCg*)
  // atomic form of Accumulate (ablation schedule LBM_SCHED_ATOMIC_A): this
  // level's contributions to the coarser level's coalescence entries,
  // grouped by the 128-cell quarter block of the contributing fine cell
  std::vector<uint32_t> sc_qoff;      // [4 nfluid + 1] CSR offsets into sc_items
  std::vector<uint32_t> sc_items;     // [n][4] {fine population index, coarse slot, |B|, 0}
  // volumetric variant: expressions are uint4 {pop index,
  // tag | nwall << 4 | wall0 << 8, wall1 | wall2 << 16, 0} (lattice.h kVt*)
  std::vector<uint32_t> vfill;        // [n][8]: {dst pop index, 0, 0, 0, expr}: the second-substep ghost packets
  std::vector<uint32_t> vavg;         // [n][36]: {slot pop index or ~0u, 0, 0, 0, 8 exprs}: coarse averages
  std::vector<uint32_t> avg_base;     // host only: [nblocks*512] first vavg entry of an averaged cell, or ~0u
  std::vector<int32_t> plain_ids;     // fluid blocks without special cells (Morton order)
  std::vector<int32_t> special_ids;   // the others (Morton order)

  // coordinate maps (cells in [0, n) per axis)
  int32_t block_at(int64_t x, int64_t y, int64_t z) const {
    return blkmap[(((x + off[0]) >> 3) * nb[1] + ((y + off[1]) >> 3)) * nb[2] + ((z + off[2]) >> 3)];
  }
  int local_at(int64_t x, int64_t y, int64_t z) const {
    return (int)(((x + off[0]) & 7) + 8 * ((y + off[1]) & 7) + 64 * ((z + off[2]) & 7));
  }
  int64_t cell_x(int32_t b, int l) const { return (int64_t)origin[3 * b] * 8 + (l & 7) - off[0]; }
  int64_t cell_y(int32_t b, int l) const { return (int64_t)origin[3 * b + 1] * 8 + ((l >> 3) & 7) - off[1]; }
  int64_t cell_z(int32_t b, int l) const { return (int64_t)origin[3 * b + 2] * 8 + (l >> 6) - off[2]; }
};

struct BuildInput {
  int32_t n0[3];
  int32_t periodic[3];
  int32_t levels;
  int32_t Q;
  const uint8_t* const* masks;
  // x-slab partition (local grid = owned slab + one coarse cell of halo on
  // each side that has a neighbour rank): owned level-0 x range [lo, hi) in
  // local coordinates (hi < 0: everything owned), and which sides have a
  // neighbour (0: -x, 1: +x)
  int32_t owned_lo0 = 0, owned_hi0 = -1;
  int32_t has_nb[2] = {0, 0};
  int32_t variant = 0;                // 0 paper's method, 1 volumetric ghost advection
  int32_t align_blocks = 1;           // choose HostLevel::off (0: block grids start at cell 0)
  int32_t block_order = 0;            // 0 Morton, 1 raster (grid_builder.cpp block_key)
};

// Returns 0 on success; otherwise an lbm_status code with `err` filled.
int build_grid(const BuildInput& in, std::vector<HostLevel>& out, std::string& err);

}  // namespace lbmr
