// level_step.cu — sm_100a kernels of the multi-level LBM hot path.
//
// F_L^k (level_step_kernel): ONE fused kernel per level-substep.  For every
// fluid leaf p of level L it pulls the Q populations of substep k
//   * Streaming, Eq.(2): same-level source p - e_q, via the 8^3 block's
//     neighbour table;
//   * Explosion, Eq.(10): source inside a coarser leaf -> that leaf's
//     post-collision value C_{L-1}^{ceil(k/2)} (reading R-A1; both fine
//     substeps read the same coarse value, R-A4; the fine level reads the
//     coarse grid directly);
//   * Coalescence, Eq.(11), gather form of Accumulate: source
//     cell refined -> (sum_B C_{L+1}^{2k-1} + sum_B C_{L+1}^{2k}) / (2|B|) over
//     the fine fluid leaves beta with beta + e_q inside p (R-A2, R-A3);
//   * bounce-back / moving wall / outflow (R-A11);
// then collides (BGK Eq.(3)/(5), or KBC [18] per R-A9) with ω_L (Eq.9) and
// writes C_L^{k+1}.  Populations are stored shifted, g = f - w (R-A16), in
// AoSoA layout [block][q][512] so every same-level pull of a warp is
// a 128-byte-coalesced row load.
//
// The CTA is half an 8^3 block (256 threads, one cell each).  Links whose
// source is not a same-level fluid leaf reachable by the block arithmetic are
// flagged per cell by the host builder (cellinfo) and resolved from
// precomputed link records in resolve_slow(); blocks without such cells (the
// bulk) never read cellinfo.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <utility>

#include "../../include/lbmr.h"
#include "kernels.h"
#include "lattice.h"

namespace lbmr {

// griddepcontrol.wait (sm_90+): block until the stream's preceding kernel
// (programmatic dependent launch) has completed and its writes are visible
__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

__constant__ int c_ex[27] = {LBMR_EX_LIST};
__constant__ int c_ey[27] = {LBMR_EY_LIST};
__constant__ int c_ez[27] = {LBMR_EZ_LIST};

template <int Q>
__device__ __forceinline__ double wq_rt(int q) {
  // runtime-q weight (slow path only)
  if (Q == 19) return q == 0 ? 1.0 / 3.0 : (q < 7 ? 1.0 / 18.0 : 1.0 / 36.0);
  return q == 0 ? 8.0 / 27.0 : (q < 7 ? 2.0 / 27.0 : (q < 19 ? 1.0 / 54.0 : 1.0 / 216.0));
}

template <typename T>
__device__ __forceinline__ T nan_of() {
  return T(NAN);
}

// ---------------------------------------------------------------- collision
// Moments of shifted populations: rho = 1 + sum g (Eq.6), j = sum e g (Eq.7).
template <int Q, typename T>
__device__ __forceinline__ void moments(const T (&g)[Q], T& drho, T& jx, T& jy, T& jz) {
  drho = T(0); jx = T(0); jy = T(0); jz = T(0);
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    drho += g[q];
    if (ex(q) > 0) jx += g[q]; else if (ex(q) < 0) jx -= g[q];
    if (ey(q) > 0) jy += g[q]; else if (ey(q) < 0) jy -= g[q];
    if (ez(q) > 0) jz += g[q]; else if (ez(q) < 0) jz -= g[q];
  }
}

// shifted equilibrium g^eq_q = w_q (drho + rho (3 e.u + 4.5 (e.u)^2 - 1.5 u^2))
template <int Q, typename T>
__device__ __forceinline__ T geq(int q, T drho, T rho, T ux, T uy, T uz, T usq15) {
  const T eu = T(ex(q)) * ux + T(ey(q)) * uy + T(ez(q)) * uz;
  return T(weight<Q>(q)) * (drho + rho * (T(3) * eu + T(4.5) * eu * eu - usq15));
}

template <typename T>
__device__ __forceinline__ T recip(T x) {
  return T(1) / x;
}
template <>
__device__ __forceinline__ float recip<float>(float x) {
  return __frcp_rn(x);  // correctly rounded, no division sequence
}

// weight class of direction q: 0 rest, 1 axis, 2 edge, 3 corner
__host__ __device__ constexpr int wclass(int q) { return q == 0 ? 0 : q < 7 ? 1 : q < 19 ? 2 : 3; }

// BGK, Eq.(3) with Eq.(5), on shifted populations, organised by opposite
// pairs (q, q+1):  ω g^eq_q = A_w + B_w (e_q.j) + C_w (e_q.j)^2 with
//   A_w = ω w (δρ - 1.5 |j|^2/ρ),  B_w = 3 ω w,  C_w = 4.5 ω w / ρ
// (ρ u = j), so the pair shares A + C (e.j)^2 and flips the sign of B (e.j).
#ifndef LBMR_BGK_ALT_FORM
#define LBMR_BGK_ALT_FORM 0
#endif
template <int Q, typename T>
__device__ __forceinline__ void collide_bgk(T (&g)[Q], T omega) {
  T drho = g[0], jx = T(0), jy = T(0), jz = T(0);
#pragma unroll
  for (int q = 1; q < Q; q += 2) {
    const T s = g[q] + g[q + 1];
    const T d = g[q] - g[q + 1];
    drho += s;
    if (ex(q) > 0) jx += d; else if (ex(q) < 0) jx -= d;
    if (ey(q) > 0) jy += d; else if (ey(q) < 0) jy -= d;
    if (ez(q) > 0) jz += d; else if (ez(q) < 0) jz -= d;
  }
  const T inv = recip<T>(T(1) + drho);
  const T jj = jx * jx + jy * jy + jz * jz;
  const T base = omega * (drho - T(1.5) * jj * inv);
  const T cfac = T(4.5) * omega * inv;
  const T bfac = T(3) * omega;
  const T omw = T(1) - omega;
  T A[4], B[4], C[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const T w = T(weight<Q>(c == 0 ? 0 : c == 1 ? 1 : c == 2 ? 7 : 19));
    A[c] = w * base;
    B[c] = w * bfac;
    C[c] = w * cfac;
  }
#if LBMR_BGK_ALT_FORM
  // diagnostic build only (tools/fp32_floor.py): the same BGK step in another
  // association, g* = g - ω (g - g^eq), to measure how far two equally valid
  // fp32 evaluations of the method drift apart
  (void)omw;
  const T iw = recip<T>(omega);
  g[0] = g[0] - omega * (g[0] - A[0] * iw);
#pragma unroll
  for (int q = 1; q < Q; q += 2) {
    T ej = T(0);
    if (ex(q) > 0) ej += jx; else if (ex(q) < 0) ej -= jx;
    if (ey(q) > 0) ej += jy; else if (ey(q) < 0) ej -= jy;
    if (ez(q) > 0) ej += jz; else if (ez(q) < 0) ej -= jz;
    const int c = wclass(q);
    const T sym = (C[c] * ej * ej + A[c]) * iw;
    const T asym = B[c] * ej * iw;
    g[q] = g[q] - omega * (g[q] - (sym + asym));
    g[q + 1] = g[q + 1] - omega * (g[q + 1] - (sym - asym));
  }
#else
  g[0] = omw * g[0] + A[0];
#pragma unroll
  for (int q = 1; q < Q; q += 2) {
    T ej = T(0);
    if (ex(q) > 0) ej += jx; else if (ex(q) < 0) ej -= jx;
    if (ey(q) > 0) ej += jy; else if (ey(q) < 0) ej -= jy;
    if (ez(q) > 0) ej += jz; else if (ez(q) < 0) ej -= jz;
    const int c = wclass(q);
    const T sym = C[c] * ej * ej + A[c];
    const T asym = B[c] * ej;
    g[q] = omw * g[q] + (sym + asym);
    g[q + 1] = omw * g[q + 1] + (sym - asym);
  }
#endif
}

template <>
__device__ __forceinline__ double recip<double>(double x) {
  return __drcp_rn(x);
}

// Opaque copy: stops the compiler from merging recomputations of g^eq in
// separate passes back into values held live across them (occupancy).
template <typename T>
__device__ __forceinline__ T fresh(T x) {
  if constexpr (sizeof(T) == 4) asm volatile("" : "+f"(x));
  else asm volatile("" : "+d"(x));
  return x;
}

// Reciprocal of a positive, normal f^eq_i inside the entropic products:
// fp32 uses the one-instruction MUFU approximation (rel. error <= 2^-23, far
// inside the fp32 parity bar); fp64 keeps the correctly rounded one.
template <typename T>
__device__ __forceinline__ T rcp_feq(T x) {
  if constexpr (sizeof(T) == 4) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
  } else {
    return __drcp_rn(x);
  }
}

// KBC (reading R-A9) on shifted populations; D3Q27 only:
//   f^neq = g - g^eq;  Δs from the deviatoric second moments of f^neq;
//   Δh = f^neq - Δs;  γ = 1/β - (2 - 1/β) <Δs|Δh>/<Δh|Δh>,  <X|Y> = Σ X Y / f^eq
//   (γ = 2 if <Δh|Δh> < 1e-30);  f* = f - β (2 Δs + γ Δh),  β = ω/2.
// Moment form: algebraically the same collision as the oracle's
// kbc_collide, organised to cut the instruction count:
//  * the second moments of f^neq come from the populations directly:
//    sum_i g_i e_ia e_ib = S_ab and sum_i g^eq_i e_ia e_ib = δρ/3 δ_ab +
//    j_a j_b/ρ (Eq.5 on a lattice with 4th-order isotropy, both D3Q19 and
//    D3Q27), so N_xz = (S_xx - S_zz) - (j_x² - j_z²)/ρ, N_yz likewise and
//    Π_ab = S_ab - j_a j_b/ρ for a != b (the δρ/3 terms cancel);
//  * g^eq is built twice (the entropic products, the update), never stored:
//    opaque copies of the moments (fresh()) keep the compiler from holding
//    27 g^eq values live between the passes (occupancy);
//  * f* = f - β(2Δs + γΔh) with Δh = f^neq - Δs is applied as
//    g* = g + A (g^eq - g) - B Δs, A = βγ, B = β(2 - γ).
// Populations are read through acc.get(q) and the results written through
// acc.put(q, v) (KbcRegs: the thread's registers).
template <typename T, typename Acc>
__device__ __forceinline__ void collide_kbc_acc(Acc& acc, T omega) {
  constexpr int Q = 27;
  T drho = acc.get(0), jx = T(0), jy = T(0), jz = T(0);
  // S_xx - S_zz and S_yy - S_zz accumulated directly: a pair with both (or
  // neither) of e_x, e_z nonzero adds nothing to S_xx - S_zz
  T dxz = T(0), dyz = T(0), sxy = T(0), sxz = T(0), syz = T(0);
#pragma unroll
  for (int q = 1; q < Q; q += 2) {
    const T gq = acc.get(q), gq1 = acc.get(q + 1);
    const T sm = gq + gq1;  // e_a e_b is even in e: pair sums
    const T df = gq - gq1;
    drho += sm;
    if (ex(q) > 0) jx += df; else if (ex(q) < 0) jx -= df;
    if (ey(q) > 0) jy += df; else if (ey(q) < 0) jy -= df;
    if (ez(q) > 0) jz += df; else if (ez(q) < 0) jz -= df;
    if (ex(q) && !ez(q)) dxz += sm; else if (!ex(q) && ez(q)) dxz -= sm;
    if (ey(q) && !ez(q)) dyz += sm; else if (!ey(q) && ez(q)) dyz -= sm;
    if (ex(q) * ey(q) > 0) sxy += sm; else if (ex(q) * ey(q) < 0) sxy -= sm;
    if (ex(q) * ez(q) > 0) sxz += sm; else if (ex(q) * ez(q) < 0) sxz -= sm;
    if (ey(q) * ez(q) > 0) syz += sm; else if (ey(q) * ez(q) < 0) syz -= sm;
  }
  const T inv = recip<T>(T(1) + drho);
  const T jxi = jx * inv, jyi = jy * inv, jzi = jz * inv;
  const T nxz = dxz - (jx * jxi - jz * jzi);
  const T nyz = dyz - (jy * jyi - jz * jzi);
  const T sixth = T(1) / T(6);
  const T sx = (T(2) * nxz - nyz) * sixth, sy = (T(2) * nyz - nxz) * sixth, sz = -(nxz + nyz) * sixth;
  const T exy = (sxy - jx * jyi) * T(0.25), exz = (sxz - jx * jzi) * T(0.25), eyz = (syz - jy * jzi) * T(0.25);
  const T base0 = drho - T(1.5) * (jx * jxi + jy * jyi + jz * jzi);  // g^eq = w (base + 3 e.j + 4.5 (e.j)^2 / ρ)
  const T c450 = T(4.5) * inv;
  auto geq_pair = [](int q, T base, T c45, T x, T y, T z, T& sym, T& asym) {
    T ej = T(0);
    if (ex(q) > 0) ej += x; else if (ex(q) < 0) ej -= x;
    if (ey(q) > 0) ej += y; else if (ey(q) < 0) ej -= y;
    if (ez(q) > 0) ej += z; else if (ez(q) < 0) ej -= z;
    const T w = T(weight<Q>(q));
    sym = w * (base + c45 * ej * ej);
    asym = (w * T(3)) * ej;
  };
  auto ds = [&](int q) -> T {
    const int n2 = ex(q) * ex(q) + ey(q) * ey(q) + ez(q) * ez(q);
    if (n2 == 1) return ex(q) ? sx : (ey(q) ? sy : sz);
    if (n2 == 2) {
      if (ez(q) == 0) return T(ex(q) * ey(q)) * exy;
      if (ey(q) == 0) return T(ex(q) * ez(q)) * exz;
      return T(ey(q) * ez(q)) * eyz;
    }
    return T(0);
  };
  // <Δs|Δh>, <Δh|Δh> with weights 1/f^eq (two partial sums each)
  T sh = 0, hh = 0, sh2 = 0, hh2 = 0;
  {
    const T base = fresh(base0), c45 = fresh(c450), x = fresh(jx), y = fresh(jy), z = fresh(jz);
    {
      const T geq0 = T(weight<Q>(0)) * base;
      const T h = acc.get(0) - geq0;
      hh += h * h * rcp_feq<T>(T(weight<Q>(0)) + geq0);
    }
#pragma unroll
    for (int q = 1; q < Q; q += 2) {
      T sym, asym;
      geq_pair(q, base, c45, x, y, z, sym, asym);
      const T a = T(weight<Q>(q)) + sym;  // f^eq = a ± asym
      T i0, i1;
      if constexpr (sizeof(T) == 4) {
        i0 = rcp_feq<T>(a + asym);
        i1 = rcp_feq<T>(a - asym);
      } else {  // one rounded reciprocal per pair: 1/(a±b) = (a∓b)/(a²-b²)
        const T r = recip<T>(a * a - asym * asym);
        i0 = (a - asym) * r;
        i1 = (a + asym) * r;
      }
      // Δs is even in e (ds(q) == ds(q + 1)) and zero on the corner
      // directions: h = (g - (g^eq_sym + Δs)) ∓ g^eq_asym, and the <Δs|Δh>
      // terms of the corners are skipped (compile time)
      const bool kHasS = ex(q) * ex(q) + ey(q) * ey(q) + ez(q) * ez(q) < 3;
      const T sq = ds(q);
      const T u = kHasS ? sym + sq : sym;
      const T h0 = (acc.get(q) - u) - asym, h1 = (acc.get(q + 1) - u) + asym;
      const T t0 = h0 * i0, t1 = h1 * i1;
      if (kHasS) {
        sh += sq * t0;
        sh2 += sq * t1;
      }
      hh += h0 * t0;
      hh2 += h1 * t1;
    }
  }
  sh += sh2;
  hh += hh2;
  const T beta = omega / T(2);
  const T gamma = (hh < T(1e-30)) ? T(2) : T(1) / beta - (T(2) - T(1) / beta) * sh / hh;
  const T A = beta * gamma, B = beta * (T(2) - gamma);
  {
    const T base = fresh(base0), c45 = fresh(c450), x = fresh(jx), y = fresh(jy), z = fresh(jz);
    {
      const T g0 = acc.get(0);
      acc.put(0, g0 + A * (T(weight<Q>(0)) * base - g0));
    }
#pragma unroll
    for (int q = 1; q < Q; q += 2) {
      T sym, asym;
      geq_pair(q, base, c45, x, y, z, sym, asym);
      const T gq = acc.get(q), gq1 = acc.get(q + 1);
      T r0 = gq + A * ((sym + asym) - gq);
      T r1 = gq1 + A * ((sym - asym) - gq1);
      if (ex(q) * ex(q) + ey(q) * ey(q) + ez(q) * ez(q) < 3) {  // Δs = 0 on corner directions
        r0 -= B * ds(q);
        r1 -= B * ds(q + 1);
      }
      acc.put(q, r0);
      acc.put(q + 1, r1);
    }
  }
}

template <typename T>
struct KbcRegs {
  T (&g)[27];
  __device__ __forceinline__ T get(int q) const { return g[q]; }
  __device__ __forceinline__ void put(int q, T v) { g[q] = v; }
};

template <typename T>
__device__ __forceinline__ void collide_kbc(T (&g)[27], T omega) {
  KbcRegs<T> a{g};
  collide_kbc_acc<T>(a, omega);
}

template <int Q, int COLL, typename T>
__device__ __forceinline__ void collide(T (&g)[Q], T omega) {
  if constexpr (COLL == LBM_KBC && Q == 27) collide_kbc<T>(g, omega);
  else collide_bgk<Q, T>(g, omega);
}

// ---------------------------------------------------------------- slow links
// A fluid leaf's links whose source is not a plain same-level neighbour were
// resolved by the host builder into records (lattice.h kLink*).  The kernel
// reads them in batches of four and issues the four source loads back to back:
//   kLinkSame / kLinkCoarse  -> one load from C_L^k / C_{L-1}^{ceil(k/2)}
//                               (Explosion, Eq.10);
//   kLinkBC / kLinkFace      -> halfway bounce-back of the cell's own
//                               post-collision opposite population, + 6 w_q
//                               e_q.u_w for a moving wall / inlet, g = 0
//                               (f = w_q) for outflow;
//   kLinkCoal                -> (sum_B C_{L+1}^{2k-1} + sum_B C_{L+1}^{2k})/(2|B|)
//                               (Coalescence, Eq.11, R-A2/R-A3), summed
//                               in candidate order like the oracle.
__device__ __forceinline__ int opp_rt(int q) { return q == 0 ? 0 : ((q & 1) ? q + 1 : q - 1); }

// Values go to this thread's column sv[q * 256] of a shared buffer
// (conflict-free for any q per lane).
template <int Q, typename T, int NT = 256>
__device__ __forceinline__ void resolve_slow_sv(const StepParams<T>& P, T* sv, uint32_t slow, unsigned j, int blk,
                                                int t) {
  const unsigned own = (unsigned)blk * (unsigned)(Q * kCells) + (unsigned)t;
#ifndef LBMR_SLOW_NB
#define LBMR_SLOW_NB 4
#endif
  constexpr int NB = (Q == 19 && sizeof(T) == 4) ? 4 : LBMR_SLOW_NB;
  while (slow) {
    int qb[NB];
    uint2 eb[NB];
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      qb[b] = -1;
      eb[b] = make_uint2(0u, 0u);
      if (slow) {
        qb[b] = __ffs(slow) - 1;
        slow &= slow - 1;
        eb[b] = __ldg(P.links + j);
        ++j;
      }
    }
    T v[NB];
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      v[b] = T(0);
      if (qb[b] >= 0) {
        const unsigned tag = eb[b].y >> 28;
        const T* base = (tag == kLinkCoarse) ? P.csrc : (tag == kLinkTemp ? P.vtemp : P.src);
        const unsigned idx =
            (tag <= kLinkCoarse || tag == kLinkTemp) ? eb[b].x : own + (unsigned)(opp_rt(qb[b]) * kCells);
        v[b] = __ldg(base + idx);
      }
    }
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      const int q = qb[b];
      if (q < 0) continue;
      const unsigned tag = eb[b].y >> 28;
      T val = v[b];
      if (tag == kLinkBC || tag == kLinkFace) {
        const unsigned cls = (tag == kLinkFace) ? (unsigned)__ldg(P.face_cls + eb[b].x) : eb[b].x;
        const int kind = __ldg(&P.bc[cls].kind);
        if (kind == LBM_BC_OUTFLOW) {
          val = T(0);
        } else if (kind == LBM_BC_VELOCITY) {
          const double eu = c_ex[q] * __ldg(&P.bc[cls].u[0]) + c_ey[q] * __ldg(&P.bc[cls].u[1]) +
                            c_ez[q] * __ldg(&P.bc[cls].u[2]);
          val += T(6.0 * wq_rt<Q>(q) * 1.0 * eu);
        }
      } else if (tag == kLinkCoal) {
        const unsigned n = eb[b].y & 0xfu;
        const uint32_t* c = P.coal + eb[b].x;
        T acc = T(0);
        for (unsigned m = 0; m < n; ++m) acc += __ldg(P.fa + __ldg(c + m));
        for (unsigned m = 0; m < n; ++m) acc += __ldg(P.fb + __ldg(c + m));
        val = acc / T(2 * n);
      }
      sv[q * NT] = val;
    }
  }
}

template <int Q, typename T, int NT = 256>
__device__ __forceinline__ void resolve_slow_links(const StepParams<T>& P, uint32_t slow, unsigned j, int blk, int t) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  resolve_slow_sv<Q, T, NT>(P, reinterpret_cast<T*>(smem_raw) + threadIdx.x, slow, j, blk, t);
}

// g[q] = this thread's column entry q for every q of the mask
template <int Q, typename T, int NT = 256>
__device__ __forceinline__ void merge_column(T (&g)[Q], uint32_t mask) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const T* sv = reinterpret_cast<const T*>(smem_raw) + threadIdx.x;
#pragma unroll
  for (int q = 1; q < Q; ++q)
    if ((mask >> q) & 1u) g[q] = sv[q * NT];
}

// ---------------------------------------------------------------- fused kernel
// Per-thread source geometry of the same-level pull inside an 8^3 block:
// the source coordinate along each axis for e = +1 / -1 / 0 and the
// neighbour-slot offset, nonzero only for a thread on the block face.
struct PullGeom {
  int xm, xp, x0, ym, yp, y0, zm, zp, z0;
  int dxm, dxp, dym, dyp, dzm, dzp;
  __device__ __forceinline__ explicit PullGeom(int t) {
    const int lx = t & 7, ly = (t >> 3) & 7, lz = t >> 6;
    x0 = lx; xm = (lx - 1) & 7; xp = (lx + 1) & 7;
    y0 = ly << 3; ym = ((ly - 1) & 7) << 3; yp = ((ly + 1) & 7) << 3;
    z0 = lz << 6; zm = ((lz - 1) & 7) << 6; zp = ((lz + 1) & 7) << 6;
    dxm = (lx == 0) ? -1 : 0; dxp = (lx == 7) ? 1 : 0;
    dym = (ly == 0) ? -3 : 0; dyp = (ly == 7) ? 3 : 0;
    dzm = (lz == 0) ? -9 : 0; dzp = (lz == 7) ? 9 : 0;
  }
  template <int q>
  __device__ __forceinline__ int local() const {
    return (ex(q) > 0 ? xm : (ex(q) < 0 ? xp : x0)) | (ey(q) > 0 ? ym : (ey(q) < 0 ? yp : y0)) |
           (ez(q) > 0 ? zm : (ez(q) < 0 ? zp : z0));
  }
  template <int q>
  __device__ __forceinline__ int slot() const {
    return 13 + (ex(q) > 0 ? dxm : (ex(q) < 0 ? dxp : 0)) + (ey(q) > 0 ? dym : (ey(q) < 0 ? dyp : 0)) +
           (ez(q) > 0 ? dzm : (ez(q) < 0 ? dzp : 0));
  }
};

// Streaming loads / stores of populations (variants selected at build time):
// LBMR_LDVAR 0 = ld.global.nc, 1 = + L2::256B prefetch, 2 = + L1::no_allocate
// + L2::256B, 3 = L1::no_allocate; LBMR_STVAR 0 = st.global, 1 = st.global.cs
// (evict-first).  Re-measured with the L2 bulk prefetch (round 2, 3 runs):
// 0 / 1 beats the round-1 choice 1 / 0 by 1.0 % on cfg5 fp32 (finest level
// 0.963 -> 0.973), 0.9 % on cfg5 fp64, 0.5 % on Tab. I s3 fp64 (cfg4 KBC
// equal): the bulk prefetch replaces the per-load 256-byte L2 prefetch hint,
// and evict-first stores leave L2 to the neighbour blocks' halo reads;
// no_allocate in L1 loses the in-CTA reuse of neighbour rows (-15 %).
#ifndef LBMR_LDVAR
#define LBMR_LDVAR 0
#endif
#ifndef LBMR_STVAR
#define LBMR_STVAR 1
#endif
template <typename T>
__device__ __forceinline__ T ld_pop(const T* p) {
#if LBMR_LDVAR == 0
  return __ldg(p);
#else
  T v;
  if constexpr (sizeof(T) == 4) {
#if LBMR_LDVAR == 1
    asm volatile("ld.global.nc.L2::256B.f32 %0, [%1];" : "=f"(v) : "l"(p));
#elif LBMR_LDVAR == 2
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.f32 %0, [%1];" : "=f"(v) : "l"(p));
#else
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
#endif
  } else {
#if LBMR_LDVAR == 1
    asm volatile("ld.global.nc.L2::256B.f64 %0, [%1];" : "=d"(v) : "l"(p));
#elif LBMR_LDVAR == 2
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.f64 %0, [%1];" : "=d"(v) : "l"(p));
#else
    asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
#endif
  }
  return v;
#endif
}

template <typename T>
__device__ __forceinline__ void st_pop(T* p, T v) {
#if LBMR_STVAR == 0
  *p = v;
#else
  __stcs(p, v);
#endif
}

// PRED = false: every link is a plain same-level pull.  PRED = true: load
// only for fluid cells and existing neighbour blocks (links flagged slow are
// loaded speculatively from the block arithmetic's source and overwritten by
// resolve_slow; the source memory always exists).
template <int Q, typename T, bool PRED, int q>
__device__ __forceinline__ void pull_one(T (&g)[Q], const T* __restrict__ src, const PullGeom& G, int rec, int blk,
                                         bool fluid) {
  constexpr unsigned FULL = 0xffffffffu;
  const int nb = (q == 0) ? blk : __shfl_sync(FULL, rec, G.slot<q>());
  const unsigned off = (unsigned)nb * (unsigned)(Q * kCells) + (unsigned)G.local<q>();
  const T* p = src + q * kCells;  // constant part folds into the load's immediate offset
  if (PRED) {
    g[q] = (fluid && nb >= 0) ? ld_pop<T>(p + off) : T(0);
  } else {
    g[q] = ld_pop<T>(p + off);
  }
}

template <int Q, typename T, bool PRED, int... qs>
__device__ __forceinline__ void pull_all(T (&g)[Q], const T* __restrict__ src, const PullGeom& G, int rec, int blk,
                                         bool fluid, std::integer_sequence<int, qs...>) {
  (pull_one<Q, T, PRED, qs>(g, src, G, rec, blk, fluid), ...);
}

// Boundary links of the cell's BC source (bounce mask): NOSLIP keeps the
// bounced value, VELOCITY adds 6 w_q rho_w e_q.u_w (rho_w = 1, R-A11),
// OUTFLOW sets f_q = w_q, i.e. g_q = 0.
// The links of the bounce mask (lattice.h cellinfo [2]) were pulled
// speculatively from the block arithmetic's source.  bounce_issue() fetches
// the cell's own post-collision opposite populations (halfway bounce-back,
// P:L264) with cp.async straight into this thread's column of the shared
// staging buffer — for every direction of the warp's bounce-mask union
// (lattice.h kBounceWords), issued before the cell's own info has arrived,
// all in flight together with the pulls and without holding registers;
// merge_column() takes the cell's own bounce links from the column and
// bounce_fix() adds the BC term.
template <int Q, typename T, int NT = 256>
__device__ __forceinline__ void bounce_issue(const StepParams<T>& P, uint32_t bounce, unsigned own) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const unsigned sv = (unsigned)__cvta_generic_to_shared(reinterpret_cast<T*>(smem_raw) + threadIdx.x);
#pragma unroll
  for (int q = 1; q < Q; ++q) {
    if ((bounce >> q) & 1u) {
      const T* a = P.src + opp(q) * kCells + own;
      asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(sv + (unsigned)(q * NT * sizeof(T))), "l"(a),
                   "n"(sizeof(T))
                   : "memory");
    }
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
}

// BC term of the bounce links: NOSLIP keeps the bounced value, VELOCITY adds
// 6 w_q rho_w e_q.u_w (rho_w = 1, R-A11), OUTFLOW sets f_q = w_q, i.e. g_q = 0.
template <int Q, typename T>
__device__ __forceinline__ void bounce_fix(const StepParams<T>& P, T (&g)[Q], uint32_t bounce, unsigned key) {
  const unsigned cls = key < kFaceSourceBase ? key : (unsigned)__ldg(P.face_cls + (key - kFaceSourceBase));
  const int kind = __ldg(&P.bc[cls].kind);
  if (kind == LBM_BC_NOSLIP) return;
  if (kind == LBM_BC_OUTFLOW) {
#pragma unroll
    for (int q = 1; q < Q; ++q)
      if ((bounce >> q) & 1u) g[q] = T(0);
    return;
  }
  const double ux = __ldg(&P.bc[cls].u[0]), uy = __ldg(&P.bc[cls].u[1]), uz = __ldg(&P.bc[cls].u[2]);
#pragma unroll
  for (int q = 1; q < Q; ++q) {
    if ((bounce >> q) & 1u) {
      const double eu = ex(q) * ux + ey(q) * uy + ez(q) * uz;
      g[q] += T(6.0 * weight<Q>(q) * 1.0 * eu);
    }
  }
}

template <int Q, typename T>
__device__ __forceinline__ void store_cell(const T (&g)[Q], T* __restrict__ dst, int blk, int t) {
  T* d = dst + (unsigned)blk * (unsigned)(Q * kCells) + t;
#pragma unroll
  for (int q = 0; q < Q; ++q) st_pop<T>(d + q * kCells, g[q]);
}

// Explosion ghosts: ghost cell g of level L holds its parent's
// C_{L-1} populations, so interface cells pull the exploded value (Eq.10)
// as a plain same-level load.  One thread per ghost; only the planes an owned
// fluid leaf pulls are refreshed (5 of 19 on a flat D3Q19 interface).
template <int Q, typename T>
__device__ __forceinline__ void ghost_fill_one(const StepParams<T>& P, int i) {
  if (i >= P.nghost) return;
  const uint32_t gc = __ldg(P.ghost_fill + 3 * i), pc = __ldg(P.ghost_fill + 3 * i + 1);
  const uint32_t mask = __ldg(P.ghost_fill + 3 * i + 2);
  T* d = P.dst + (gc >> 9) * (unsigned)(Q * kCells) + (gc & 511u);
  const T* s = P.gsrc + (pc >> 9) * (unsigned)(Q * kCells) + (pc & 511u);
  if (mask & kGhostRowOwn) {
    // the ghost is the row's only live cell: store the value over the whole
    // 8-cell row (aligned full sectors; the other seven cells are never read)
    T* r = d - (gc & 7u);
#pragma unroll
    for (int q = 1; q < Q; ++q)
      if ((mask >> q) & 1u) {
        const T v = __ldg(s + q * kCells);
        if constexpr (sizeof(T) == 4) {
          float4* w = reinterpret_cast<float4*>(r + q * kCells);
          w[0] = w[1] = make_float4(v, v, v, v);
        } else {
          double2* w = reinterpret_cast<double2*>(r + q * kCells);
          w[0] = w[1] = w[2] = w[3] = make_double2(v, v);
        }
      }
    return;
  }
#pragma unroll
  for (int q = 1; q < Q; ++q)
    if ((mask >> q) & 1u) d[q * kCells] = __ldg(s + q * kCells);
}

__host__ __device__ constexpr int ghost_ctas(int n) { return (n + 255) / 256; }
__host__ __device__ constexpr int halo_fill_ctas(int n) { return (n + kHaloCtaThreads - 1) / kHaloCtaThreads; }

// Volumetric variant: one gather expression = a population of
// buffer A, B or C (tag) followed by up to three wall reflections, innermost
// first (halfway bounce-back as the oracle's wall_value: NOSLIP keeps the
// value, VELOCITY adds 6 w_d e_d.u_w, OUTFLOW gives f = w, i.e. g = 0).
template <int Q, typename T>
__device__ __forceinline__ T vexpr(const uint32_t* e, const T* A, const T* B, const T* C, const BCEntry* bc,
                                   const uint8_t* face_cls) {
  const uint32_t tag = e[1] & 15u, nw = (e[1] >> 4) & 3u;
  T v = T(0);
  if (tag == kVtA) v = A[e[0]];
  else if (tag == kVtB) v = B[e[0]];
  else if (tag == kVtC) v = C[e[0]];
  for (uint32_t w = 0; w < nw; ++w) {
    const uint32_t wd = w == 0 ? (e[1] >> 8) & 0x3fffu : (w == 1 ? e[2] & 0xffffu : e[2] >> 16);
    const uint32_t src = wd & 511u, dir = wd >> 9;
    const unsigned cls = src < kFaceSourceBase ? src : (unsigned)__ldg(face_cls + (src - kFaceSourceBase));
    const int kind = __ldg(&bc[cls].kind);
    if (kind == LBM_BC_OUTFLOW) {
      v = T(0);
    } else if (kind == LBM_BC_VELOCITY) {
      const double eu = c_ex[dir] * __ldg(&bc[cls].u[0]) + c_ey[dir] * __ldg(&bc[cls].u[1]) +
                        c_ez[dir] * __ldg(&bc[cls].u[2]);
      v += T(6.0 * wq_rt<Q>(dir) * 1.0 * eu);
    }
  }
  return v;
}

// Trailing CTAs of a level kernel: refresh the ghosts the next kernel of this
// level pulls — parent copies (Eq.10), or in the volumetric variant's second
// substep the advected packets.
template <int Q, typename T>
__device__ __forceinline__ void trail_fill(const StepParams<T>& P, int i) {
#ifdef LBMR_DEBUG_NOFILL
  return;  // timing experiment only (wrong results)
#endif
  ghost_fill_one<Q, T>(P, i);
  if (i < P.nvfill) {
    const uint32_t* e = P.vfill + 8 * (size_t)i;
    P.dst[e[0]] = vexpr<Q, T>(e + 4, P.src, P.gsrc, nullptr, P.bc, P.face_cls);
  }
  // ablation schedule LBM_SCHED_ATOMIC_A: reset the accumulators (coalescence
  // ghost slots) the next fine collisions add into ("it will reset the
  // ghost layer")
  if (i < P.nzero) P.dst[__ldg(P.zero_list + i)] = T(0);
}

__host__ __device__ inline int trail_items(int nghost, int nvfill) { return nghost > nvfill ? nghost : nvfill; }
template <typename T>
__host__ __device__ inline int trail_count(const StepParams<T>& p) {
  const int a = trail_items(p.nghost, p.nvfill);
  return a > p.nzero ? a : p.nzero;
}

// Ablation schedule LBM_SCHED_ATOMIC_A (Fig. 4c, the paper's Accumulate as a
// scatter atomic write fused into the Collision): the CTA that
// just stored the post-collision values of cells [base, base + NT) of block
// blk adds each value a coarse coalescence link needs into that link's
// accumulator (the coarse ghost slot), v / (2|B|) when the division is fused
// (no O kernel) or v.  Items are grouped per 128-cell quarter block, so a CTA
// reads only values its own threads wrote (visible after the barrier).  At
// most 8 fine cells add into one accumulator, so contention is low.
template <typename T, int NT>
__device__ __forceinline__ void accumulate_scatter(const StepParams<T>& P, int blk, int base) {
  const unsigned q0 = (unsigned)blk * 4u + (unsigned)(base >> 7);
  const unsigned a = __ldg(P.sc_qoff + q0), b = __ldg(P.sc_qoff + q0 + NT / 128);
  if (a == b) return;  // CTA-uniform
  __syncthreads();
  for (unsigned i = a + threadIdx.x; i < b; i += NT) {
    const uint4 it = __ldg(P.sc_items + i);
    T v = P.dst[it.x];
    if (P.sc_scaled) v = v / T(2 * it.z);
    atomicAdd(P.acc + it.y, v);
  }
}

// Minimum resident CTAs per SM (register budget 65536 / (256 * MINB)),
// chosen per variant from ptxas -v and measurement.
// D3Q19 fp32: 5 units = 48 registers (round 2, with the L2 prefetch and the
// in-record PDL gate: cfg5 +1.4 %, cfg3 +1.9 %, uniform512 +1.1 % over 6
// units = 40 registers; round 1 without the prefetch measured 6 better)
#ifndef LBMR_OCC_Q19F
#define LBMR_OCC_Q19F 5
#endif
#ifndef LBMR_OCC_KBCF
#define LBMR_OCC_KBCF 4
#endif
#ifndef LBMR_OCC_KBCD
#define LBMR_OCC_KBCD 2
#endif
#ifndef LBMR_OCC_BGKD
#define LBMR_OCC_BGKD 3
#endif
template <int Q, typename T, int COLL = LBM_BGK>
struct PlainOcc {
  static constexpr int value = COLL == LBM_KBC ? (sizeof(T) == 4 ? LBMR_OCC_KBCF : LBMR_OCC_KBCD)
                               : (Q == 19 && sizeof(T) == 4) ? LBMR_OCC_Q19F
                               : (sizeof(T) == 4 ? 3 : (Q == 19 ? LBMR_OCC_BGKD : 2));
};

// ---------------------------------------------------------------- halo protocol
// x-slab partition.  Blocks holding an owned cell of a cut
// plane are stored (and launched) first.  Their CTAs (a) wait until every
// neighbour rank has finished the cut-plane part of all previous kernels
// (its bumps of our flag reach our kernel count), (b) store their cut-plane
// cells' post-collision populations straight into the neighbour's halo cells
// (peer memory: CUDA IPC over NVLink, or another grid on the same device),
// and (c) the last of them bumps the neighbours' flags.  Interior CTAs never
// wait.  Only cut-plane cells read halo cells, so this orders every halo read
// after the matching write and every overwrite after the previous read.
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

template <typename T>
__device__ __forceinline__ void halo_signal(const StepParams<T>& P, int nproto) {
  // the barrier orders every thread's halo stores before thread 0's
  // system-scope fence (fences are cumulative), which orders them before the
  // count: one fence per CTA instead of one per thread
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();
    if (atomicAdd(P.flags + 3, 1ull) == (unsigned long long)(nproto - 1)) {
      P.flags[3] = 0ull;
      P.flags[2] += 1ull;
      __threadfence_system();
      for (int s = 0; s < 2; ++s)
        if (P.has_nb[s]) atomicAdd_system(P.peer_flag[s], 1ull);
    }
  }
}

template <int Q, typename T>
__device__ __forceinline__ void halo_store(const StepParams<T>& P, const T (&g)[Q], int blk, int t) {
  if (blk >= P.nboundary) return;
#pragma unroll
  for (int s = 0; s < 2; ++s) {
    if (!P.has_nb[s]) continue;
    const int i = __ldg(P.bpeer + ((unsigned)blk * 2 + s) * kCells + t);
    if (i < 0) continue;
    const unsigned pc = __ldg(P.peer_cells[s] + i);
    T* d = P.peer_dst[s] + (pc >> 9) * (unsigned)(Q * kCells) + (pc & 511u);
#pragma unroll
    for (int q = 0; q < Q; ++q) d[q * kCells] = g[q];
  }
}

// ---------------------------------------------------------------- fused kernel
// One cell of F_L^k (all fluid blocks in storage = Morton order, cut-plane
// blocks first).  CTA = half an 8^3 block, one cell per thread.  No shared
// memory and no barrier: each warp reads its block's record (27 neighbour
// ids, special slot, origin, per-warp fluid and slow-link masks) with one
// coalesced and two broadcast loads and picks neighbour ids with
// __shfl_sync.  A warp whose 32 cells are fluid leaves with only same-level
// links (the bulk) takes the predicate-free pull; the test is warp-uniform.
// Other warps load the same way for their fluid cells, and the few cells with
// slow links then apply their link records.  Offsets are 32-bit
// (host-checked: nblocks * Q * 512 < 2^32).
// COLLIDE = false: the stream-only half S_L^k of the unfused schedule
// (lbm_set_schedule): the pulled post-streaming populations are stored as is.
// Bounce copies issued with the pulls (per-warp union masks, lattice.h
// kBounceWords) or after the cell's info: measured per lattice — D3Q27
// (cfg4: every warp walls) +3 % BGK, +20 % KBC; D3Q19 (cfg5) -0.4 %.
#ifndef LBMR_EARLY_BOUNCE_Q19
#define LBMR_EARLY_BOUNCE_Q19 0
#endif
template <int Q>
constexpr bool kEarlyBounce = (Q == 27) || LBMR_EARLY_BOUNCE_Q19;

// Coalescence fused into the coarse level kernel (schedule
// LBM_SCHED_CTA_GATHER): before its cells need them, the CTA evaluates the Eq.11
// gathers (R-A2/R-A3) of its own fluid leaves' coalescence links,
// units [a, e) of P.cg_*.  Four lanes per unit: lane m loads candidate slot m
// of C_{L+1}^{2k-1} (fa) and of C_{L+1}^{2k} (fb); the group's first lane
// adds the values through __shfl_sync in the oracle's order (fa over the
// slots, then fb; a |B| > 4 entry spans the next group too), divides by 2|B|
// and writes the result into the destination cell's column of the shared
// staging buffer and its direction bit into the cell's mask; the cell takes
// it after its pulls (coal_merge) like a record value.  Runs at the CTA's
// start, before the populations are live in registers (no spills), U units
// per group in flight together.  Same terms in the same order as the gather
// kernel (coalesce_one): bitwise equal to the gather schedule.
#ifndef LBMR_CG_UNROLL
#define LBMR_CG_UNROLL 4
#endif
template <typename T, int NT>
__device__ __forceinline__ void coal_fused(const StepParams<T>& P, uint32_t* cmask, unsigned a, unsigned e) {
  constexpr unsigned FULL = 0xffffffffu;
  constexpr int U = LBMR_CG_UNROLL, G = NT / 4;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* col = reinterpret_cast<T*>(smem_raw);
  cmask[threadIdx.x] = 0u;
  __syncthreads();
  const int lane = threadIdx.x & 31, gl = lane & ~3, m = lane & 3;
  for (unsigned base = a; base < e; base += G * U) {  // CTA-uniform trip count
    uint32_t c[U], d[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const unsigned u = base + (unsigned)(j * G) + (threadIdx.x >> 2);
      const bool in = u < e;
      c[j] = in ? __ldg(P.cg_cand + 4 * u + m) : ~0u;
      d[j] = in ? __ldg(P.cg_dest + u) : (kCgSkip << 12);
    }
    T va[U], vb[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      va[j] = c[j] != ~0u ? __ldg(P.fa + c[j]) : T(0);
      vb[j] = c[j] != ~0u ? __ldg(P.fb + c[j]) : T(0);
    }
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const unsigned kind = d[j] >> 12;
      const unsigned vm = (__ballot_sync(FULL, c[j] != ~0u) >> gl) & (kind == kCgPair ? 0xffu : 0xfu);
      T acc = T(0);
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const T v = __shfl_sync(FULL, va[j], gl + i);
        if ((vm >> i) & 1u) acc += v;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const T v = __shfl_sync(FULL, vb[j], gl + i);
        if ((vm >> i) & 1u) acc += v;
      }
      if (m == 0 && kind != kCgSkip && vm) {
        const unsigned t = d[j] & 127u, q = (d[j] >> 7) & 31u;
        col[q * NT + t] = acc / T(2 * __popc(vm));
        atomicOr(&cmask[t], 1u << q);
      }
    }
  }
  __syncthreads();
}

template <int Q, typename T, int NT>
__device__ __forceinline__ void coal_merge(T (&g)[Q], const uint32_t* cmask) {
  const uint32_t cm = cmask[threadIdx.x];
  if (cm) merge_column<Q, T, NT>(g, cm);
}

// CG: the CTA gathers its cells' coalescence links itself (P.cg_*; level
// kernels of the CTA_GATHER schedule only: the product's kernels are compiled
// without this code, so their register assignment is untouched)
template <int Q, int COLL, typename T, bool HALO, bool COLLIDE = true, int NT = 256, bool CG = false>
__device__ __forceinline__ void step_cell(const StepParams<T>& P, int blk, int t, bool pdl_gate = false) {
  constexpr unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int* R = P.nbr + blk * kRec;
  const int rec = __ldg(R + lane);
  const uint32_t fm = (uint32_t)__ldg(R + kRecFluid + (t >> 5));
  const uint32_t sm = (uint32_t)__ldg(R + kRecSpecial + (t >> 5));
  // fused coalescence: this quarter-block CTA's gather units (CTA-uniform),
  // evaluated first (one program point for the whole CTA: barriers inside)
  __shared__ uint32_t cmask[NT];
  unsigned ca = 0u, ce = 0u;
  if constexpr (CG && NT == 128) {
    if (P.cg_qoff) {
      const unsigned cta = (unsigned)blk * 4u + (unsigned)(t >> 7);
      ca = __ldg(P.cg_qoff + cta);
      ce = __ldg(P.cg_qoff + cta + 1);
      if (ca < ce) coal_fused<T, NT>(P, cmask, ca, ce);
    }
  }
  // PDL after the coalescence gather: a warp whose block pulls coalescence
  // ghosts waits for the gather before its pulls (the flag rides in the
  // record the warp has just loaded: no extra round trip)
  if (pdl_gate && __shfl_sync(FULL, rec, kRecCoalPull) != 0) griddep_wait();
  const PullGeom G(t);
  T g[Q];
  const unsigned own = (unsigned)blk * (unsigned)(Q * kCells) + (unsigned)t;
  // KBC: one collision / store site for both paths (half the code: fewer
  // instruction-cache misses with the long collision); BGK: separate sites,
  // so the plain path keeps its own spill-free register assignment
  constexpr bool kShared = (COLL == LBM_KBC);
#ifdef LBMR_DEBUG_ALLPLAIN
  const bool plain = true;  // timing experiment only (wrong results): every warp takes the plain path
#else
  const bool plain = (fm == FULL && sm == 0u);  // warp-uniform
#endif
  int slot = 0;
  bool fluid = true, special = false;
  uint32_t bm = 0u;
  uint4 ci = make_uint4(0u, 0u, 0u, kNoBCSource);
  uint32_t cm = 0u;  // coalescence links of the cell (special path)
  if (plain) {
    pull_all<Q, T, false>(g, P.src, G, rec, blk, true, std::make_integer_sequence<int, Q>{});
    // the cell's coalescence links from the column (merged in each path:
    // a common merge point would join the plain path's register assignment
    // with the special path's)
    if (CG && ca < ce) coal_merge<Q, T, NT>(g, cmask);
  } else {
    slot = __shfl_sync(FULL, rec, kRecSlot);
    fluid = (fm >> lane) & 1u;
    special = (sm >> lane) & 1u;
    if constexpr (kEarlyBounce<Q>) {
      // bounce-back sources (the cell's own opposite populations) of every
      // direction some cell of this warp bounces: copied into the thread's
      // shared-memory column right after the pulls, not after the cell's
      // info arrives (partly fluid warps without special cells skip the
      // load: sm is warp-uniform)
      bm = (sm != 0u && fluid) ? __ldg(P.bmask + (unsigned)slot * kBounceWords + (t >> 5)) : 0u;
    } else {
      // the cell's info first, its bounce copies once it has arrived
      if (special) ci = __ldg(P.cellinfo + (unsigned)slot * kCells + t);
    }
    pull_all<Q, T, true>(g, P.src, G, rec, blk, fluid, std::make_integer_sequence<int, Q>{});
    // the cell's coalescence links join its record merge below (never
    // bounce or record links; the warp-union bounce copies skip them)
    if (CG && ca < ce) cm = cmask[threadIdx.x];
  }
  if (plain) {
    if (!kShared) {
      if (COLLIDE) collide<Q, COLL, T>(g, P.omega);
      store_cell<Q, T>(g, P.dst, blk, t);
      if (HALO) halo_store<Q, T>(P, g, blk, t);
      return;
    }
  } else {
    if constexpr (kEarlyBounce<Q>) {
#ifndef LBMR_DEBUG_NOSLOW
      if (bm & ~cm) bounce_issue<Q, T, NT>(P, bm & ~cm, own);
#endif
      if (!fluid) return;
      if (special) ci = __ldg(P.cellinfo + (unsigned)slot * kCells + t);
#ifndef LBMR_DEBUG_NOSLOW
      if (bm & ~cm) asm volatile("cp.async.wait_all;" ::: "memory");
      const uint32_t recs = ci.x & ((1u << Q) - 1u);
      if (recs) resolve_slow_links<Q, T, NT>(P, recs, ci.y, blk, t);  // into the column, disjoint from ci.z
      if (ci.z | recs | cm) merge_column<Q, T, NT>(g, ci.z | recs | cm);
      if (ci.z) bounce_fix<Q, T>(P, g, ci.z, ci.w);
#endif
    } else {
      if (!fluid) return;
#ifndef LBMR_DEBUG_NOSLOW
      if (ci.z) {
        bounce_issue<Q, T, NT>(P, ci.z, own);
        asm volatile("cp.async.wait_all;" ::: "memory");
        merge_column<Q, T, NT>(g, ci.z);
        bounce_fix<Q, T>(P, g, ci.z, ci.w);
      }
      const uint32_t recs = ci.x & ((1u << Q) - 1u);
      if (recs | cm) {
        if (recs) resolve_slow_links<Q, T, NT>(P, recs, ci.y, blk, t);
        merge_column<Q, T, NT>(g, recs | cm);
      }
#endif
    }
  }
  if (COLLIDE) collide<Q, COLL, T>(g, P.omega);
  store_cell<Q, T>(g, P.dst, blk, t);
  if (HALO) halo_store<Q, T>(P, g, blk, t);
}

// Prologue C_L^1: collision of the initial state.  INPLACE: the collide-only
// half C_L^{k+1} of the unfused schedule, src == dst (each thread reads its
// own cell before overwriting it, so plain loads instead of ld.global.nc).
template <int Q, int COLL, typename T, bool HALO, bool INPLACE = false>
__device__ __forceinline__ void collide_cell(const StepParams<T>& P, int blk, int t) {
  const uint32_t fm = (uint32_t)__ldg(P.nbr + blk * kRec + kRecFluid + (t >> 5));
  if (!((fm >> (threadIdx.x & 31)) & 1u)) return;
  T g[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const T* a = P.src + ((unsigned)blk * Q + q) * kCells + t;
    g[q] = INPLACE ? *a : __ldg(a);
  }
  collide<Q, COLL, T>(g, P.omega);
  store_cell<Q, T>(g, P.dst, blk, t);
  if (HALO) halo_store<Q, T>(P, g, blk, t);
}

// CTA size of the fused single-rank kernel per variant: a quarter of an 8^3
// block (128 threads) instead of a half (256); the CTAs per SM scale so the
// register budget (PlainOcc, in 256-thread units) is unchanged.  The finer
// CTA granularity measured +1.5-2 % on cfg5 / cfg3 / uniform512 (D3Q19), +5-6 %
// on the D3Q27 KBC / BGK workloads (fewer warps idle behind a CTA's slowest
// warp at the end of its life, more CTAs in flight per SM).
#ifndef LBMR_NT_KBCD
#define LBMR_NT_KBCD 128
#endif
#ifndef LBMR_NT_OTHER
#define LBMR_NT_OTHER 128
#endif
template <int Q, int COLL, typename T>
struct StepCta {
  static constexpr int threads = (COLL == LBM_KBC && sizeof(T) == 8) ? LBMR_NT_KBCD : LBMR_NT_OTHER;
  static constexpr int per_block = kCells / threads;
  static constexpr int min_blocks = (PlainOcc<Q, T, COLL>::value * 256) / threads;
};

// L2 prefetch (P.prefetch blocks ahead in storage order): the first CTA of a
// block has one thread ask the TMA unit (cp.async.bulk.prefetch.L2, SASS
// UBLKPF) to bring the populations of block blk + prefetch — contiguous, Q x
// 512 values — into L2, so the CTAs that process that block shortly after
// pull from L2 instead of DRAM.  The resident warps' registers bound the
// loads in flight; the bulk prefetch adds memory-level parallelism without
// registers.  Measured (16 blocks ahead): cfg5 fp32 +3 %, fp64 +3 % (finest
// level 0.954 -> 0.978 of the copy peak), Tab. I s3 fp64 KBC +10 % (0.77 ->
// 0.85), cfg4 KBC fp32 +8 % (0.72 -> 0.78); 512 blocks ahead thrashes L2.
template <int Q, typename T>
__device__ __forceinline__ void prefetch_block(const StepParams<T>& P, int blk) {
  if (P.prefetch <= 0 || threadIdx.x != 0) return;
  const int pb = blk + P.prefetch;
  if (pb >= P.nfluid) return;
  const T* a = P.src + (size_t)pb * (Q * kCells);
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"((unsigned)(Q * kCells * sizeof(T)))
               : "memory");
}

// Programmatic dependent launch (sm_90+): wait until the preceding kernel of
// the stream (the coalescence gather) has completed and its writes are
// visible; let the following kernel launch early.
__device__ __forceinline__ void pdl_wait() { griddep_wait(); }
__device__ __forceinline__ void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;" :::); }

template <int Q, int COLL, typename T, bool CG = false>
__global__ void __launch_bounds__(StepCta<Q, COLL, T>::threads, StepCta<Q, COLL, T>::min_blocks)
    level_step_all(const StepParams<T> P) {
  constexpr int NT = StepCta<Q, COLL, T>::threads, PB = StepCta<Q, COLL, T>::per_block;
  const int main = P.nfluid * PB;
  // PDL chain (P.pdl_chain): launched as the programmatic dependent of the
  // previous level kernel, so this grid's CTAs become resident during that
  // kernel's tail; they wait for its completion before touching memory and
  // then let the next kernel launch.  After the coalescence gather (P.pdl)
  // only the CTAs that pull its ghosts wait first, the others after their
  // work; either way the kernel completes only after its predecessor.
  if (P.pdl_chain && !P.pdl) pdl_wait();
  if ((int)blockIdx.x >= main) {  // trailing CTAs refresh the explosion ghosts
    if (P.pdl || P.pdl_chain) pdl_launch_dependents();
    trail_fill<Q, T>(P, ((int)blockIdx.x - main) * NT + threadIdx.x);
    if (P.pdl) pdl_wait();  // this kernel completes only after the gather
    return;
  }
  const int b = (int)blockIdx.x;
  if ((b % PB) == 0) prefetch_block<Q, T>(P, b / PB);
  if (P.pdl || P.pdl_chain) pdl_launch_dependents();
  // under PDL the gather may still be running: warps whose block pulls a
  // coalescence ghost wait for it before their pulls (inside step_cell), all
  // others after their work (a second wait returns at once)
  step_cell<Q, COLL, T, false, true, NT, CG>(P, b / PB, (b % PB) * NT + threadIdx.x, P.pdl != 0);
  if (P.sc_qoff) accumulate_scatter<T, NT>(P, b / PB, (b % PB) * NT);
  if (P.pdl) pdl_wait();
}

// Partitioned variant: grid = 4 * max(nfluid, 1) quarter-block CTAs; the first nbctas run
// the halo protocol around their work.
// One thread waits until every neighbour has completed the cut-plane part of
// all kernels this rank has completed (its bumps of our flag reach our
// kernel count).  A separate one-CTA launch, so that no CTA of a level kernel
// ever spins: partitions emulated on one device cannot starve each other.
// The spin is bounded: a neighbour that never arrives (a rank that died or
// stopped stepping) turns into a device trap after kHaloWaitTimeoutNs instead
// of a hung GPU, so the caller's next synchronising call reports LBM_E_CUDA.
#ifndef LBMR_HALO_WAIT_TIMEOUT_S
#define LBMR_HALO_WAIT_TIMEOUT_S 120
#endif
constexpr unsigned long long kHaloWaitTimeoutNs = (unsigned long long)LBMR_HALO_WAIT_TIMEOUT_S * 1000000000ull;

__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ void halo_spin_wait(const unsigned long long* flags, int nb0, int nb1) {
  const unsigned long long mine = *(volatile const unsigned long long*)(flags + 2);
  const unsigned long long t0 = globaltimer_ns();
  for (int s = 0; s < 2; ++s) {
    if (!(s == 0 ? nb0 : nb1)) continue;
    while (ld_acquire_sys(flags + s) < mine) {
      __nanosleep(256);
      if (globaltimer_ns() - t0 > kHaloWaitTimeoutNs) {
        printf("lbmr: halo wait timed out (side %d: %llu of %llu kernels)\n", s, ld_acquire_sys(flags + s), mine);
        __trap();
      }
    }
  }
}

__global__ void halo_wait_kernel(const unsigned long long* flags, int nb0, int nb1) {
  halo_spin_wait(flags, nb0, nb1);
}

// In-kernel form (P.halo_spin, set when every neighbour rank is on another
// GPU): only the CTAs that read halo cells or store into the neighbour (the
// protocol CTAs) wait, thread 0 spinning and the CTA's barrier ordering the
// other threads' reads after its acquire.  Saves the one-thread wait kernel
// and its graph-node gap before every level kernel.  Not used when ranks
// share a GPU: there, spinning CTAs could hold every SM slot while the kernel
// they wait for has none.
__device__ __forceinline__ void halo_spin_cta(const unsigned long long* flags, int nb0, int nb1) {
  if (threadIdx.x == 0) halo_spin_wait(flags, nb0, nb1);
  __syncthreads();
}

template <int Q, int COLL, typename T, bool STREAM>
__global__ void __launch_bounds__(kHaloCtaThreads, (PlainOcc<Q, T, COLL>::value * 256) / kHaloCtaThreads)
    level_step_halo(const StepParams<T> P) {
  constexpr int NT = kHaloCtaThreads, PB = kHaloCtasPerBlock;
  // CTA order: the cut-plane CTAs [0, nbctas) (blocks stored first), then the
  // ghost-refresh CTAs, then the interior CTAs.  Both protocol groups sit at
  // the front, so the completion signal (their last CTA) fires early in the
  // kernel and a neighbour's next kernel waits for this kernel's cut-plane
  // part only, not for its end (ranks stay loosely coupled: one kernel of
  // slack instead of lockstep).
  const int nfill = halo_fill_ctas(trail_count(P));
  const int bid = (int)blockIdx.x;
  const bool fill = bid >= P.nbctas && bid < P.nbctas + nfill;
  const int mb = bid < P.nbctas ? bid : bid - nfill;  // main CTA index (interior CTAs after the fills)
  const int blk = mb / PB;
  const int t = (mb % PB) * NT + threadIdx.x;
  // the wait happened in halo_wait_kernel just before this launch; cut-plane
  // CTAs (which write the neighbour's halo) and ghost-refresh CTAs (which may
  // read L-1 halo cells) count towards this kernel's completion signal
  const bool proto = bid < P.nbctas || fill;
  if (P.pdl_chain) {  // PDL chain: resident during the previous kernel's tail (see level_step_all)
    pdl_wait();
    pdl_launch_dependents();
  }
  if (P.halo_spin && proto) halo_spin_cta(P.flags, P.has_nb[0], P.has_nb[1]);
  if (!fill && (mb % PB) == 0) prefetch_block<Q, T>(P, blk);
  if (fill) {
    trail_fill<Q, T>(P, (bid - P.nbctas) * NT + threadIdx.x);
  } else if (blk < P.nfluid) {
    if (STREAM) step_cell<Q, COLL, T, true, true, NT>(P, blk, t);
    else collide_cell<Q, COLL, T, true>(P, blk, t);
  }
  if (proto) halo_signal<T>(P, P.nbctas + nfill);
}

template <int Q, int COLL, typename T>
__global__ void __launch_bounds__(256) level_collide(const StepParams<T> P) {
  if ((int)blockIdx.x >= 2 * P.nfluid) {
    trail_fill<Q, T>(P, ((int)blockIdx.x - 2 * P.nfluid) * 256 + threadIdx.x);
    return;
  }
  collide_cell<Q, COLL, T, false>(P, blockIdx.x >> 1, ((blockIdx.x & 1) << 8) | threadIdx.x);
  if (P.sc_qoff) accumulate_scatter<T, 256>(P, blockIdx.x >> 1, (blockIdx.x & 1) << 8);
}

// Unfused schedule (fusion ablation, Fig.4 / Fig.9): S_L^k pulls
// (streaming, Explosion ghosts, Coalescence ghosts, BC) into dst without
// colliding; C_L^{k+1} then collides dst in place.  Same arithmetic as the
// fused F_L^k, so the result is bitwise identical; it moves 4Q values per
// leaf instead of 2Q.
template <int Q, typename T>
__global__ void __launch_bounds__(256, PlainOcc<Q, T, LBM_BGK>::value) level_stream(const StepParams<T> P) {
  const int main = 2 * P.nfluid;
  if ((int)blockIdx.x >= main) {
    trail_fill<Q, T>(P, ((int)blockIdx.x - main) * 256 + threadIdx.x);
    return;
  }
  step_cell<Q, LBM_BGK, T, false, false>(P, blockIdx.x >> 1, ((blockIdx.x & 1) << 8) | threadIdx.x);
}

template <int Q, int COLL, typename T>
__global__ void __launch_bounds__(256) level_collide_inplace(const StepParams<T> P) {
  collide_cell<Q, COLL, T, false, true>(P, blockIdx.x >> 1, ((blockIdx.x & 1) << 8) | threadIdx.x);
  if (P.sc_qoff) accumulate_scatter<T, 256>(P, blockIdx.x >> 1, (blockIdx.x & 1) << 8);
}

// Ablation schedule LBM_SCHED_SPLIT_E: Explosion (Eq.10) as its own kernel,
// refreshing the explosion ghosts of dst from the parent level's
// post-collision state gsrc right before the level's streaming kernel.
template <int Q, typename T>
__global__ void __launch_bounds__(256) explosion_refresh(const StepParams<T> P) {
  ghost_fill_one<Q, T>(P, (int)blockIdx.x * 256 + threadIdx.x);
}

// ---------------------------------------------------------------- init / macroscopic
template <int Q, typename T>
__global__ void __launch_bounds__(512) init_eq_kernel(T* pop, const uint8_t* types, const double* rho,
                                                      const double* u) {
  const int blk = blockIdx.x, t = threadIdx.x;
  const size_t c = (size_t)blk * kCells + t;
  T* d = pop + (size_t)blk * Q * kCells + t;
  if (types[c] != kFluid) {
#pragma unroll
    for (int q = 0; q < Q; ++q) d[(size_t)q * kCells] = T(0);
    return;
  }
  const double r = rho[c], ux = u[3 * c], uy = u[3 * c + 1], uz = u[3 * c + 2];
  const double usq15 = 1.5 * (ux * ux + uy * uy + uz * uz);
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const double eu = ex(q) * ux + ey(q) * uy + ez(q) * uz;
    // Eq.(5) minus w_q:  w_q (rho - 1 + rho (3 eu + 4.5 eu^2 - 1.5 u^2))
    d[(size_t)q * kCells] = T(weight<Q>(q) * ((r - 1.0) + r * (3.0 * eu + 4.5 * eu * eu - usq15)));
  }
}

template <int Q, typename T>
__global__ void __launch_bounds__(512) macroscopic_kernel(const T* pop, const int32_t* rec, double* rho, double* u,
                                                          double* block_mass) {
  const int blk = blockIdx.x, t = threadIdx.x;
  const size_t c = (size_t)blk * kCells + t;
  double r = 0.0;
  const uint32_t fm = (uint32_t)rec[blk * kRec + kRecFluid + (t >> 5)];
  const bool fluid = (fm >> (t & 31)) & 1u;  // owned fluid leaf
  if (fluid) {
    const T* s = pop + (size_t)blk * Q * kCells + t;
    double d = 0, jx = 0, jy = 0, jz = 0;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const double g = (double)s[(size_t)q * kCells];
      d += g;
      jx += ex(q) * g;
      jy += ey(q) * g;
      jz += ez(q) * g;
    }
    r = 1.0 + d;
    if (rho) rho[c] = r;
    if (u) { u[3 * c] = jx / r; u[3 * c + 1] = jy / r; u[3 * c + 2] = jz / r; }
  } else {
    if (rho) rho[c] = NAN;
    if (u) u[3 * c] = u[3 * c + 1] = u[3 * c + 2] = NAN;
  }
  if (block_mass) {
    __shared__ double sm[16];
    double v = r;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((t & 31) == 0) sm[t >> 5] = v;
    __syncthreads();
    if (t == 0) {
      double a = 0;
      for (int i = 0; i < 16; ++i) a += sm[i];
      block_mass[blk] = a;
    }
  }
}

// Probes: rho, u (Eq.6-7) of n cells given by their population cell index
// block*512 + local (or -1 -> NaN).  One thread per probe.
template <int Q, typename T>
__global__ void __launch_bounds__(256) probe_kernel(const T* __restrict__ pop, const int64_t* __restrict__ cell,
                                                    int64_t n, double* __restrict__ rho, double* __restrict__ u) {
  const int64_t i = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (i >= n) return;
  const int64_t c = cell[i];
  if (c < 0) {
    rho[i] = u[3 * i] = u[3 * i + 1] = u[3 * i + 2] = NAN;
    return;
  }
  const T* s = pop + (c >> 9) * (int64_t)(Q * kCells) + (c & 511);
  double d = 0, jx = 0, jy = 0, jz = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const double g = (double)s[(int64_t)q * kCells];
    d += g;
    jx += ex(q) * g;
    jy += ey(q) * g;
    jz += ez(q) * g;
  }
  const double r = 1.0 + d;
  rho[i] = r;
  u[3 * i] = jx / r;
  u[3 * i + 1] = jy / r;
  u[3 * i + 2] = jz / r;
}

void launch_probe(int Q, int precision, const void* pop, const int64_t* cell, int64_t n, double* rho, double* u,
                  cudaStream_t s) {
  if (n <= 0) return;
  const unsigned grid = (unsigned)((n + 255) / 256);
  if (precision == LBM_FP32) {
    if (Q == 19) probe_kernel<19, float><<<grid, 256, 0, s>>>((const float*)pop, cell, n, rho, u);
    else probe_kernel<27, float><<<grid, 256, 0, s>>>((const float*)pop, cell, n, rho, u);
  } else {
    if (Q == 19) probe_kernel<19, double><<<grid, 256, 0, s>>>((const double*)pop, cell, n, rho, u);
    else probe_kernel<27, double><<<grid, 256, 0, s>>>((const double*)pop, cell, n, rho, u);
  }
}

// Coalescence ghosts: one thread per (ghost cell, q) entry,
// entries ordered by (q, ghost) so a warp reads neighbouring fine cells of one
// plane; candidate slots structure-of-arrays (grid_builder.h coal_cand).
// Fine candidates summed in candidate order, first substep then second, like
// the oracle (Eq.11, n = 2|B|, R-A2/R-A3).
// mode: kCoalFromDst / kCoalDivide (kernels.h); fa / fb may be NULL.  The
// terms are added in the oracle's order (fa candidates, then fb candidates),
// so the split Accumulate kernels of the ablation schedules reproduce the
// one-kernel gather bitwise.
template <typename T, int K>
__device__ __forceinline__ void coalesce_one(const T* __restrict__ fa, const T* __restrict__ fb, T* dst, uint32_t d,
                                             const uint32_t* __restrict__ cand, int64_t stride, int mode) {
  uint32_t c[K];
#pragma unroll
  for (int m = 0; m < K; ++m) c[m] = __ldg(cand + m * stride);
  T acc = (mode & kCoalFromDst) ? dst[d] : T(0);
  unsigned cnt = 0;
#pragma unroll
  for (int m = 0; m < K; ++m)
    if (c[m] != ~0u) {
      if (fa) acc += __ldg(fa + c[m]);
      ++cnt;
    }
  if (fb) {
#pragma unroll
    for (int m = 0; m < K; ++m)
      if (c[m] != ~0u) acc += __ldg(fb + c[m]);
  }
  dst[d] = (mode & kCoalDivide) ? acc / T(2 * cnt) : acc;
}

template <typename T>
__global__ void __launch_bounds__(256) coalesce_kernel(const T* __restrict__ fa, const T* __restrict__ fb, T* dst,
                                                       const uint32_t* __restrict__ fill,
                                                       const uint32_t* __restrict__ cand, int64_t nmain, int64_t novf,
                                                       int mode, const unsigned long long* spin_flags, int nb0,
                                                       int nb1, int pdl_chain) {
  if (pdl_chain) pdl_wait();  // launched as the PDL dependent of the previous level kernel
  pdl_launch_dependents();    // the level kernel after it may start (it waits where it needs us)
  // partitioned grid on distinct GPUs: the candidates may be halo cells of the
  // finer level, written by the neighbour's last fine kernel
  if (spin_flags) halo_spin_cta(spin_flags, nb0, nb1);
  const int64_t i = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (i < nmain) {
    coalesce_one<T, kCoalSlots>(fa, fb, dst, __ldg(fill + i), cand + i, nmain, mode);
  } else if (i < nmain + novf) {
    const int64_t j = i - nmain;
    coalesce_one<T, kCoalSlotsMax>(fa, fb, dst, __ldg(fill + i), cand + kCoalSlots * nmain + j, novf, mode);
  }
}

// Warp-cooperative form of the gather (launch_coalesce_warp): four lanes per
// 4-slot unit, lane m loading candidate slot m of fa and fb (one coalesced
// 16-byte unit load per four lanes); the unit's first lane adds the values
// through __shfl_sync in the oracle's order (fa slots then fb slots; a pair
// spans the next unit too), like coalesce_one.
template <typename T>
__global__ void __launch_bounds__(256) coalesce_warp_kernel(const T* __restrict__ fa, const T* __restrict__ fb,
                                                            T* dst, const uint32_t* __restrict__ cand,
                                                            const uint32_t* __restrict__ udst, int64_t n, int64_t pair,
                                                            int mode, const unsigned long long* spin_flags, int nb0,
                                                            int nb1, int pdl_chain) {
  constexpr unsigned FULL = 0xffffffffu;
  if (pdl_chain) pdl_wait();
  pdl_launch_dependents();
  if (spin_flags) halo_spin_cta(spin_flags, nb0, nb1);
  const int64_t u = (int64_t)blockIdx.x * 64 + (threadIdx.x >> 2);
  const int lane = threadIdx.x & 31, gl = lane & ~3, m = lane & 3;
  const bool in = u < n;
  const uint32_t c = in ? __ldg(cand + 4 * u + m) : ~0u;
  uint32_t d = ~0u;
  if (in && m == 0) d = __ldg(udst + u);
  const T va = (fa && c != ~0u) ? __ldg(fa + c) : T(0);
  const T vb = (fb && c != ~0u) ? __ldg(fb + c) : T(0);
  const T v0 = (in && m == 0 && d != ~0u && (mode & kCoalFromDst)) ? dst[d] : T(0);
  const unsigned vm = (__ballot_sync(FULL, c != ~0u) >> gl) & (u >= pair ? 0xffu : 0xfu);
  T acc = v0;
  if (fa) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const T v = __shfl_sync(FULL, va, gl + i);
      if ((vm >> i) & 1u) acc += v;
    }
  }
  if (fb) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const T v = __shfl_sync(FULL, vb, gl + i);
      if ((vm >> i) & 1u) acc += v;
    }
  }
  if (m == 0 && d != ~0u) dst[d] = (mode & kCoalDivide) ? acc / T(2 * __popc(vm)) : acc;
}

template <int Q, typename T>
__global__ void __launch_bounds__(256) vavg_gather(const uint32_t* __restrict__ ent, int n, const T* A, const T* B,
                                                   const T* C, const BCEntry* bc, const uint8_t* face_cls, T* tmp) {
  const int i = blockIdx.x * 256 + threadIdx.x;
  if (i >= n) return;
  const uint32_t* e = ent + 36 * (size_t)i;
  T acc = T(0);
#pragma unroll
  for (int m = 0; m < 8; ++m) acc += vexpr<Q, T>(e + 4 + 4 * m, A, B, C, bc, face_cls);
  tmp[i] = acc / T(8);
}

template <typename T>
__global__ void __launch_bounds__(256) vavg_scatter(const uint32_t* __restrict__ ent, int n, const T* tmp, T* A) {
  const int i = blockIdx.x * 256 + threadIdx.x;
  if (i >= n) return;
  const uint32_t slot = __ldg(ent + 36 * (size_t)i);
  if (slot != ~0u) A[slot] = tmp[i];
}

template <int Q, typename T>
static void vavg_typed(const uint32_t* ent, int32_t n, void* A, const void* B, const void* C, const BCEntry* bc,
                       const uint8_t* fc, void* tmp, cudaStream_t s) {
  const int grid = (n + 255) / 256;
  vavg_gather<Q, T><<<grid, 256, 0, s>>>(ent, n, (const T*)A, (const T*)B, (const T*)C, bc, fc, (T*)tmp);
  vavg_scatter<T><<<grid, 256, 0, s>>>(ent, n, (const T*)tmp, (T*)A);
}

void launch_vavg(int Q, int precision, const uint32_t* ent, int32_t n, void* A, const void* B, const void* C,
                 const BCEntry* bc, const uint8_t* face_cls, void* tmp, cudaStream_t s) {
  if (n <= 0) return;
  if (precision == LBM_FP32) {
    if (Q == 19) vavg_typed<19, float>(ent, n, A, B, C, bc, face_cls, tmp, s);
    else vavg_typed<27, float>(ent, n, A, B, C, bc, face_cls, tmp, s);
  } else {
    if (Q == 19) vavg_typed<19, double>(ent, n, A, B, C, bc, face_cls, tmp, s);
    else vavg_typed<27, double>(ent, n, A, B, C, bc, face_cls, tmp, s);
  }
}

__global__ void bc_update_kernel(BCEntry* bc, int cls, BCEntry e, uint8_t* face_cls, FaceTable ft) {
  if (threadIdx.x == 0) bc[cls] = e;
  if (threadIdx.x < 27) face_cls[threadIdx.x] = ft.cls[threadIdx.x];
}

void launch_bc_update(BCEntry* bc, int cls, BCEntry e, uint8_t* face_cls, FaceTable ft, cudaStream_t s) {
  bc_update_kernel<<<1, 32, 0, s>>>(bc, cls, e, face_cls, ft);
}

// Profiling stamp (lbm_profile_step): one thread writes the device global
// timer (ns) into out[idx]; as a graph kernel node between two level kernels
// it runs after the first has completed and before the second starts.
__global__ void stamp_kernel(unsigned long long* out, int idx) { out[idx] = globaltimer_ns(); }

void launch_stamp(unsigned long long* out, int idx, cudaStream_t s) { stamp_kernel<<<1, 1, 0, s>>>(out, idx); }

void launch_halo_wait(const unsigned long long* flags, int nb0, int nb1, cudaStream_t s) {
  halo_wait_kernel<<<1, 1, 0, s>>>(flags, nb0, nb1);
}

// cudaLaunchKernelEx with the programmatic-stream-serialization attribute
// (pdl = 1) or a plain launch
template <typename Kern, typename... Args>
static void launch_maybe_pdl(bool pdl, Kern kernel, dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                             Args... args) {
  if (!pdl) {
    kernel<<<grid, block, smem, s>>>(args...);
    return;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, kernel, args...);
}

void launch_coalesce(int Q, int precision, const void* fa, const void* fb, void* dst, const uint32_t* fill,
                     const uint32_t* cand, int64_t n_main, int64_t n_ovf, int mode, cudaStream_t s,
                     const unsigned long long* spin_flags, int nb0, int nb1, int pdl_chain) {
  (void)Q;
  const int64_t n = n_main + n_ovf;
  if (n <= 0) return;
  const unsigned grid = (unsigned)((n + 255) / 256);
  if (precision == LBM_FP32)
    launch_maybe_pdl(pdl_chain != 0, coalesce_kernel<float>, dim3(grid), dim3(256), 0, s, (const float*)fa,
                     (const float*)fb, (float*)dst, fill, cand, n_main, n_ovf, mode, spin_flags, nb0, nb1, pdl_chain);
  else
    launch_maybe_pdl(pdl_chain != 0, coalesce_kernel<double>, dim3(grid), dim3(256), 0, s, (const double*)fa,
                     (const double*)fb, (double*)dst, fill, cand, n_main, n_ovf, mode, spin_flags, nb0, nb1,
                     pdl_chain);
}

void launch_coalesce_warp(int precision, const void* fa, const void* fb, void* dst, const uint32_t* cand,
                          const uint32_t* udst, int64_t n_units, int64_t pair, int mode, cudaStream_t s,
                          const unsigned long long* spin_flags, int nb0, int nb1, int pdl_chain) {
  if (n_units <= 0) return;
  const unsigned grid = (unsigned)((n_units + 63) / 64);
  if (precision == LBM_FP32)
    launch_maybe_pdl(pdl_chain != 0, coalesce_warp_kernel<float>, dim3(grid), dim3(256), 0, s, (const float*)fa,
                     (const float*)fb, (float*)dst, cand, udst, n_units, pair, mode, spin_flags, nb0, nb1, pdl_chain);
  else
    launch_maybe_pdl(pdl_chain != 0, coalesce_warp_kernel<double>, dim3(grid), dim3(256), 0, s, (const double*)fa,
                     (const double*)fb, (double*)dst, cand, udst, n_units, pair, mode, spin_flags, nb0, nb1,
                     pdl_chain);
}

// ---------------------------------------------------------------- dispatch
// dynamic shared memory of the stepping kernels: the slow-link staging
// buffer sv[Q][256] of resolve_slow
template <int Q, typename T>
constexpr size_t slow_smem() { return (size_t)Q * 256 * sizeof(T); }

template <int Q, int COLL, typename T>
static void launch_typed(int kind, const void* params, cudaStream_t s) {
  const StepParams<T>& p = *static_cast<const StepParams<T>*>(params);
  dim3 block(256);
  const size_t sm = slow_smem<Q, T>();
  const int gc = ghost_ctas(trail_count(p));
  if (kind == 5) {  // Explosion only (ablation E kernel)
    if (p.nghost > 0) explosion_refresh<Q, T><<<dim3(ghost_ctas(p.nghost)), block, 0, s>>>(p);
    return;
  }
  if (p.nbctas > 0) {  // partitioned: always launched (the protocol must run)
    if (!p.halo_spin) halo_wait_kernel<<<1, 1, 0, s>>>(p.flags, p.has_nb[0], p.has_nb[1]);
    dim3 grid(kHaloCtasPerBlock * std::max(p.nfluid, 1) + halo_fill_ctas(trail_count(p)));
    const size_t hs = (size_t)Q * kHaloCtaThreads * sizeof(T);
    if (kind == 1) level_step_halo<Q, COLL, T, false><<<grid, dim3(kHaloCtaThreads), 0, s>>>(p);
    else launch_maybe_pdl(p.pdl_chain != 0, level_step_halo<Q, COLL, T, true>, grid, dim3(kHaloCtaThreads), hs, s, p);
    return;
  }
  if (p.nfluid <= 0 && trail_count(p) <= 0) return;
  if (kind == 1) {
    level_collide<Q, COLL, T><<<dim3(2 * p.nfluid + gc), block, 0, s>>>(p);
  } else if (kind == 3) {
    level_stream<Q, T><<<dim3(2 * p.nfluid + gc), block, sm, s>>>(p);
  } else if (kind == 4) {
    if (p.nfluid > 0) level_collide_inplace<Q, COLL, T><<<dim3(2 * p.nfluid), block, 0, s>>>(p);
  } else {
    constexpr int NT = StepCta<Q, COLL, T>::threads;
    const int gct = (trail_count(p) + NT - 1) / NT;
    const dim3 grid(p.nfluid * StepCta<Q, COLL, T>::per_block + gct), blk(NT);
    const size_t smem = (size_t)Q * NT * sizeof(T);
    if (p.cg_qoff) launch_maybe_pdl(p.pdl || p.pdl_chain, level_step_all<Q, COLL, T, true>, grid, blk, smem, s, p);
    else launch_maybe_pdl(p.pdl || p.pdl_chain, level_step_all<Q, COLL, T>, grid, blk, smem, s, p);
  }
}

// Load every kernel of the library now.  With lazy module loading (the CUDA
// 12 default) the first launch of a function can wait for the device to go
// idle, which deadlocks against a partition's spinning halo CTAs waiting for
// a neighbour grid whose kernels this host thread has not launched yet.
template <int Q, int COLL, typename T>
static void preload_variant() {
  cudaFuncSetAttribute(level_step_all<Q, COLL, T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)slow_smem<Q, T>());
  cudaFuncSetAttribute(level_step_all<Q, COLL, T, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)slow_smem<Q, T>());
  cudaFuncSetAttribute(level_step_halo<Q, COLL, T, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       (int)slow_smem<Q, T>());
  cudaFuncSetAttribute(level_stream<Q, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)slow_smem<Q, T>());
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, level_stream<Q, T>);
  cudaFuncGetAttributes(&a, level_collide_inplace<Q, COLL, T>);
  cudaFuncGetAttributes(&a, level_step_all<Q, COLL, T>);
  cudaFuncGetAttributes(&a, level_step_all<Q, COLL, T, true>);
  cudaFuncGetAttributes(&a, level_collide<Q, COLL, T>);
  cudaFuncGetAttributes(&a, level_step_halo<Q, COLL, T, true>);
  cudaFuncGetAttributes(&a, level_step_halo<Q, COLL, T, false>);
  cudaFuncGetAttributes(&a, explosion_refresh<Q, T>);
}

void preload_kernels() {
  preload_variant<19, LBM_BGK, float>();
  preload_variant<27, LBM_BGK, float>();
  preload_variant<27, LBM_KBC, float>();
  preload_variant<19, LBM_BGK, double>();
  preload_variant<27, LBM_BGK, double>();
  preload_variant<27, LBM_KBC, double>();
  cudaFuncAttributes a;
  cudaFuncGetAttributes(&a, halo_wait_kernel);
  cudaFuncGetAttributes(&a, stamp_kernel);
  cudaFuncGetAttributes(&a, bc_update_kernel);
  cudaFuncGetAttributes(&a, coalesce_kernel<float>);
  cudaFuncGetAttributes(&a, probe_kernel<19, float>);
  cudaFuncGetAttributes(&a, vavg_gather<19, float>);
  cudaFuncGetAttributes(&a, vavg_gather<27, float>);
  cudaFuncGetAttributes(&a, vavg_gather<19, double>);
  cudaFuncGetAttributes(&a, vavg_gather<27, double>);
  cudaFuncGetAttributes(&a, vavg_scatter<float>);
  cudaFuncGetAttributes(&a, vavg_scatter<double>);
  cudaFuncGetAttributes(&a, probe_kernel<27, float>);
  cudaFuncGetAttributes(&a, probe_kernel<19, double>);
  cudaFuncGetAttributes(&a, probe_kernel<27, double>);
  cudaFuncGetAttributes(&a, coalesce_kernel<double>);
  cudaFuncGetAttributes(&a, coalesce_warp_kernel<float>);
  cudaFuncGetAttributes(&a, coalesce_warp_kernel<double>);
  cudaFuncGetAttributes(&a, init_eq_kernel<19, float>);
  cudaFuncGetAttributes(&a, init_eq_kernel<27, float>);
  cudaFuncGetAttributes(&a, init_eq_kernel<19, double>);
  cudaFuncGetAttributes(&a, init_eq_kernel<27, double>);
  cudaFuncGetAttributes(&a, macroscopic_kernel<19, float>);
  cudaFuncGetAttributes(&a, macroscopic_kernel<27, float>);
  cudaFuncGetAttributes(&a, macroscopic_kernel<19, double>);
  cudaFuncGetAttributes(&a, macroscopic_kernel<27, double>);
}

void launch_level_step(int Q, int collision, int precision, int kind, const void* params, cudaStream_t s) {
  if (precision == LBM_FP32) {
    if (Q == 19) launch_typed<19, LBM_BGK, float>(kind, params, s);
    else if (collision == LBM_KBC) launch_typed<27, LBM_KBC, float>(kind, params, s);
    else launch_typed<27, LBM_BGK, float>(kind, params, s);
  } else {
    if (Q == 19) launch_typed<19, LBM_BGK, double>(kind, params, s);
    else if (collision == LBM_KBC) launch_typed<27, LBM_KBC, double>(kind, params, s);
    else launch_typed<27, LBM_BGK, double>(kind, params, s);
  }
}

void launch_init_eq(int Q, int precision, void* pop, const uint8_t* types, int32_t nfluid, const double* rho,
                    const double* u, cudaStream_t s) {
  if (nfluid <= 0) return;
  if (precision == LBM_FP32) {
    if (Q == 19) init_eq_kernel<19, float><<<nfluid, 512, 0, s>>>((float*)pop, types, rho, u);
    else init_eq_kernel<27, float><<<nfluid, 512, 0, s>>>((float*)pop, types, rho, u);
  } else {
    if (Q == 19) init_eq_kernel<19, double><<<nfluid, 512, 0, s>>>((double*)pop, types, rho, u);
    else init_eq_kernel<27, double><<<nfluid, 512, 0, s>>>((double*)pop, types, rho, u);
  }
}

void launch_macroscopic(int Q, int precision, const void* pop, const int32_t* rec, int32_t nblk, double* rho,
                        double* u, double* block_mass, cudaStream_t s) {
  if (nblk <= 0) return;
  if (precision == LBM_FP32) {
    if (Q == 19) macroscopic_kernel<19, float><<<nblk, 512, 0, s>>>((const float*)pop, rec, rho, u, block_mass);
    else macroscopic_kernel<27, float><<<nblk, 512, 0, s>>>((const float*)pop, rec, rho, u, block_mass);
  } else {
    if (Q == 19) macroscopic_kernel<19, double><<<nblk, 512, 0, s>>>((const double*)pop, rec, rho, u, block_mass);
    else macroscopic_kernel<27, double><<<nblk, 512, 0, s>>>((const double*)pop, rec, rho, u, block_mass);
  }
}

}  // namespace lbmr
