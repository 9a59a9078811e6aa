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
  int32_t nb[3] = {0, 0, 0};     // blocks per axis (ceil(n/8))
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
  std::vector<uint32_t> cellinfo;     // [nspecial*512][2]: {bit q = slow link q, bit31 = fluid leaf;
                                      //  index of the cell's first slow-link record}
  std::vector<uint32_t> links;        // [nlinks][2] slow-link records (lattice.h kLink*)
  std::vector<uint32_t> coal;         // coalescence candidate population indices
  int64_t nlinks = 0;
  std::vector<int32_t> plain_ids;     // fluid blocks without special cells (Morton order)
  std::vector<int32_t> special_ids;   // the others (Morton order)
};

struct BuildInput {
  int32_t n0[3];
  int32_t periodic[3];
  int32_t levels;
  int32_t Q;
  const uint8_t* const* masks;
};

// Returns 0 on success; otherwise an lbm_status code with `err` filled.
int build_grid(const BuildInput& in, std::vector<HostLevel>& out, std::string& err);

}  // namespace lbmr
