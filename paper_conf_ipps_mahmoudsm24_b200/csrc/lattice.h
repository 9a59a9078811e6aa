// lattice.h — D3Q19 / D3Q27 velocity sets of the product path (host + device).
// P:L37 §II names the lattices; weights are the standard ones (Krüger et al.,
// ref [2] of the paper).  Ordering: rest, then opposite pairs (q, q+1) with
// q odd, so opp(q) = q + 1 for odd q and q - 1 for even q > 0.  D3Q19 is the
// 19-entry prefix of D3Q27.
#pragma once

#ifdef __CUDACC__
#define LBM_HD __host__ __device__
#else
#define LBM_HD
#endif

namespace lbmr {

// e_x, e_y, e_z of each direction (the lists are reused for __constant__ copies)
#define LBMR_EX_LIST 0, 1, -1, 0, 0, 0, 0, 1, -1, 1, -1, 1, -1, 1, -1, 0, 0, 0, 0, 1, -1, 1, -1, 1, -1, -1, 1
#define LBMR_EY_LIST 0, 0, 0, 1, -1, 0, 0, 1, -1, -1, 1, 0, 0, 0, 0, 1, -1, 1, -1, 1, -1, 1, -1, -1, 1, 1, -1
#define LBMR_EZ_LIST 0, 0, 0, 0, 0, 1, -1, 0, 0, 0, 0, 1, -1, -1, 1, 1, -1, -1, 1, 1, -1, -1, 1, 1, -1, 1, -1
constexpr int kEx[27] = {LBMR_EX_LIST};
constexpr int kEy[27] = {LBMR_EY_LIST};
constexpr int kEz[27] = {LBMR_EZ_LIST};

// compile-time accessors (fold to constants inside unrolled loops)
LBM_HD constexpr int ex(int q) { constexpr int t[27] = {LBMR_EX_LIST}; return t[q]; }
LBM_HD constexpr int ey(int q) { constexpr int t[27] = {LBMR_EY_LIST}; return t[q]; }
LBM_HD constexpr int ez(int q) { constexpr int t[27] = {LBMR_EZ_LIST}; return t[q]; }

LBM_HD constexpr int opp(int q) { return q == 0 ? 0 : ((q & 1) ? q + 1 : q - 1); }

template <int Q>
LBM_HD constexpr double weight(int q) {
  return Q == 19 ? (q == 0 ? 1.0 / 3.0 : q < 7 ? 1.0 / 18.0 : 1.0 / 36.0)
                 : (q == 0 ? 8.0 / 27.0 : q < 7 ? 2.0 / 27.0 : q < 19 ? 1.0 / 54.0 : 1.0 / 216.0);
}

// neighbour-block slot of an offset (dx,dy,dz) in {-1,0,1}^3
LBM_HD constexpr int nbr_slot(int dx, int dy, int dz) { return (dx + 1) + 3 * (dy + 1) + 9 * (dz + 1); }

constexpr int kBlock = 8;            // B = 8 (B compile time)
constexpr int kCells = 512;          // B^3
constexpr unsigned kFluidBit = 1u << 31;
// per-fluid-block record of 64 int32 (two 128-byte lines, one warp load
// each): [0..26] neighbour block ids by nbr_slot (-1: none, outside, or a
// block without fluid leaves), [27] special slot (-1 plain), [28..30] block
// coordinates, [31] 1 if a fluid leaf of the block pulls a coalescence ghost
// (waits for the gather kernel under programmatic dependent launch),
// [32+w] fluid-leaf mask of warp w (cells 32w..32w+31),
// [48+w] mask of the fluid leaves of warp w that have a slow link
constexpr int kRec = 64;
constexpr int kRecSlot = 27;
constexpr int kRecOrigin = 28;
constexpr int kRecCoalPull = 31;
constexpr int kRecFluid = 32;
constexpr int kRecSpecial = 48;
// per special block: 16 words, word w = union over the fluid leaves of warp w
// of their bounce masks (cellinfo [2]); the kernel issues the bounce-back
// copies for these directions before the cell's own info has arrived
constexpr int kBounceWords = 16;

// per-cell info of a special block (uint4):
//  [0] bit q = link q resolved through a slow-link record, bit 31 = fluid leaf
//  [1] index of the cell's first slow-link record
//  [2] bounce mask: bit q = link q is a boundary link of the cell's BC source
//      (halfway bounce-back of the cell's own opposite population, + the
//      moving-wall term for VELOCITY, 0 (f = w) for OUTFLOW), handled inline
//  [3] BC source: a BC class id (< 256), kFaceSourceBase + outside pattern
//      (class from the face table), or kNoBCSource
constexpr int kCellInfoWords = 4;
constexpr unsigned kFaceSourceBase = 256;
constexpr unsigned kNoBCSource = 0xffffffffu;

// slow-link record {w0, w1}: tag = w1 >> 28
//  kLinkSame   w0 = population index at level L (irregular same-level source)
//  kLinkCoarse w0 = population index at level L-1 (Explosion, Eq.10)
//  kLinkBC     w0 = BC class of the source leaf
//  kLinkFace   w0 = outside pattern (ox+1)+3(oy+1)+9(oz+1) -> class via face table
//  kLinkCoal   w0 = first index in the coalescence list, w1 & 0xf = |B|
//  kLinkTemp   w0 = index into the level's volumetric averages
constexpr unsigned kLinkSame = 0, kLinkCoarse = 1, kLinkBC = 2, kLinkFace = 3, kLinkCoal = 4, kLinkTemp = 5;

// explosion-ghost fill entry {ghost cell, parent cell, mask}: bit 31 of the
// mask = the ghost is the only live cell of its 8-cell x-row (whole-row store)
constexpr unsigned kGhostRowOwn = 1u << 31;

// volumetric-variant expression tags (which buffer the population index is in)
//  fill list of level L (run by F_L^{k-1}):  kVtA = C_L^{k-1}, kVtB = C_{L-1}
//  average list of level L (before F_L^k):   kVtA = C_L^k, kVtB = C_{L+1}^{2k-1}, kVtC = C_{L+1}^{2k}
// walls: 14 bits each, BC source (class < 256 or kFaceSourceBase + pattern)
// | direction << 9, applied innermost first
constexpr unsigned kVtNone = 0, kVtA = 1, kVtB = 2, kVtC = 3;

// coalescence gather (Eq.11): candidate slots per entry.  |B| <= 4 on every
// link of a planar interface; at most 7 of the 8 candidates 2p - e_q + c lie
// outside the coarse leaf p (the one inside is ABSENT), so 7 bounds |B|.
constexpr uint32_t kCoalSlots = 4, kCoalSlotsMax = 7;
// fused coalescence units (grid_builder.h cg_dest): kind = dest >> 12
//  kCgSingle  an entry with |B| <= 4 (its 4 slots)
//  kCgPair    the first unit of an entry with |B| > 4 (slots 0..3; 4..6 in the next unit)
//  kCgSkip    the second unit of a pair, or padding
constexpr uint32_t kCgSingle = 0, kCgPair = 1, kCgSkip = 2;

// cell type codes stored per block (mask codes + derived states)
constexpr unsigned char kAbsent = 0;    // covered by a coarser leaf, or outside the domain
constexpr unsigned char kFluid = 1;
constexpr unsigned char kRefined = 255; // covered by finer leaves
// 2..254: boundary-condition leaf of that class

}  // namespace lbmr
