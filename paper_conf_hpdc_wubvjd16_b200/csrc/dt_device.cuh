// dt_device.cuh — device-side building blocks of the pack/unpack engine, shared
// by the standalone kernels (dt_kernels.cu) and the pipelined transfer kernel
// (dt_xfer.cu).  Everything here moves bytes with integer vector types.
//
//   position resolve: stream byte p -> element e = p / tsize
//     (fast division), block b = upper_bound(boff, p mod tsize) (32-ary warp
//     search) and the element displacement by mixed radix over the levels;
//   seg_range  (S5/S6 long runs): a warp walks block segments of its slice and
//     copies each with coalesced vectors and head/tail peeling;
//   word_range (S5/S6 short blocks): each thread assembles one 16-byte vector of
//     the packed stream from G-byte words located through a shared-memory word
//     table of the template.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "dt_internal.h"

namespace dt {

// q = floor(n/d) via a 64x64 high multiply by m = floor((2^64-1)/d) and one
// correction step (the estimate is q or q-1 for every 64-bit n).
struct FastDiv {
  uint64_t d, m;
};
static inline FastDiv make_fd(uint64_t d) { return FastDiv{d, d ? ~0ull / d : 0ull}; }
__device__ __forceinline__ uint64_t fdiv(uint64_t n, const FastDiv& f) {
  uint64_t q = __umul64hi(n, f.m);
  if (n - q * f.d >= f.d) q++;
  return q;
}

// Parameters of one pack or unpack over a committed descriptor.
struct KP {
  const uint8_t* nc;  // non-contiguous origin (pack: source, unpack: destination)
  uint8_t* c;         // packed stream buffer; c[0] <-> stream byte pos
  int64_t pos, len;
  int64_t tsize, nblocks;
  const int64_t* bd;
  const int64_t* bl;
  const int64_t* boff;
  int64_t bd0, bl0;  // single-block template
  int32_t nlev;
  int32_t nwords;    // word-table entries (short kernel)
  int64_t cnt[kMaxLevels];
  int64_t stride[kMaxLevels];
  const int64_t* table[kMaxLevels];
  FastDiv fcnt[kMaxLevels];
  FastDiv ftsize;
  FastDiv fnb;  // division by nblocks (short-block window kernel)
  int64_t per_warp;
  const int32_t* wtab;
  // compact block descriptors (block-span kernel): block i = (len << 32) | (uint32)(disp
  // - wbase[i / 32]); 8 bytes per block instead of 16 (nullptr: use bd/bl)
  const uint64_t* sdesc;
  const int64_t* wbase;
};

// byte displacement of element e: mixed radix over the levels, last fastest
__device__ __forceinline__ int64_t elem_disp(const KP& P, uint64_t e) {
  int64_t disp = 0;
#pragma unroll
  for (int l = kMaxLevels - 1; l >= 0; --l) {
    if (l < P.nlev) {
      uint64_t i;
      if (l == 0) {
        i = e;
      } else {
        uint64_t q = fdiv(e, P.fcnt[l]);
        i = e - q * (uint64_t)P.cnt[l];
        e = q;
      }
      disp += P.table[l] ? __ldg(P.table[l] + i) : (int64_t)i * P.stride[l];
    }
  }
  return disp;
}

// ---------------------------------------------------------------- loads/stores
// Load policy: LD_CS streams (evict-first); LD_CG bypasses L1 (for ring slots a
// peer rewrites while this kernel runs).
enum { LD_CS = 0, LD_CG = 1 };
template <int POL, typename V>
__device__ __forceinline__ V ldv(const V* p) {
  if (POL == LD_CG) return __ldcg(p);
  return __ldcs(p);
}
#ifndef DT_STORE_WB
#define DT_STORE_WB 0
#endif
template <typename V>
__device__ __forceinline__ void stv(V* p, const V& v) {
  if (DT_STORE_WB) *p = v;  // write-back (L2-allocating) stores
  else __stcs(p, v);        // streaming (evict-first) stores
}

// Copy n bytes with the whole warp, vector width V chosen from the relative
// alignment of src and dst; head bytes peel dst to V alignment, tail bytes
// follow (the paper's prologue/middle/epilogue, [L16:c3618 §3.1]).
template <int POL, typename V, int U>
__device__ __forceinline__ void warp_copy_v(uint8_t* __restrict__ dst, const uint8_t* __restrict__ src, int64_t n,
                                            int lane) {
  constexpr int W = sizeof(V);
  int64_t head = (int64_t)((0 - (uintptr_t)dst) & (W - 1));
  if (head > n) head = n;
  const int64_t nv = (n - head) / W;
  const int64_t tail = n - head - nv * W;
  // head and tail bytes are loaded up front so that a short segment costs one
  // memory round trip (their stores happen after the body's loads are issued)
  const uint8_t hb = lane < head ? src[lane] : 0;
  const uint8_t tb = lane < tail ? src[head + nv * W + lane] : 0;
  V* d = reinterpret_cast<V*>(dst + head);
  const V* s = reinterpret_cast<const V*>(src + head);
  int64_t i = lane;
  for (; i + 32 * (U - 1) < nv; i += 32 * U) {
    V v[U];
#pragma unroll
    for (int u = 0; u < U; u++) v[u] = ldv<POL>(s + i + 32 * u);
#pragma unroll
    for (int u = 0; u < U; u++) stv(d + i + 32 * u, v[u]);
  }
  if (i < nv) {  // remainder: one predicated batch, all loads in flight together
    V v[U];
#pragma unroll
    for (int u = 0; u < U; u++) v[u] = ldv<POL>(s + min(i + 32 * u, nv - 1));
#pragma unroll
    for (int u = 0; u < U; u++)
      if (i + 32 * u < nv) stv(d + i + 32 * u, v[u]);
  }
  if (lane < head) dst[lane] = hb;
  if (lane < tail) dst[head + nv * W + lane] = tb;
}

// 16 output bytes = bytes [R, R+16) of the 32-byte window a|b (R = 1..15).
template <int R>
__device__ __forceinline__ uint4 realign(const uint4& a, const uint4& b) {
  const unsigned w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
  constexpr int ws = R / 4, bs = R % 4;
  uint4 o;
  if (bs == 0) {
    o.x = w[ws]; o.y = w[ws + 1]; o.z = w[ws + 2]; o.w = w[ws + 3];
  } else {
    o.x = __funnelshift_r(w[ws], w[ws + 1], 8 * bs);
    o.y = __funnelshift_r(w[ws + 1], w[ws + 2], 8 * bs);
    o.z = __funnelshift_r(w[ws + 2], w[ws + 3], 8 * bs);
    o.w = __funnelshift_r(w[ws + 3], w[ws + 4], 8 * bs);
  }
  return o;
}

// Relatively misaligned copy with full 16-byte accesses on both sides: the
// destination is peeled to 16 B, the source is read as aligned 16-byte vectors
// A_i, and output vector i = bytes [R, R+16) of A_i|A_{i+1}; A_{i+1} comes from
// the neighbouring lane by warp shuffle (lane 31 takes lane 0's next vector), so
// every source byte is loaded once.  R = (src - dst) mod 16 is a template
// parameter: the word-aligned cases need 1-3 shuffles per vector, none of the
// byte juggling of the paper's 8-byte prologue/epilogue scheme.
template <int POL, int R, int U>
__device__ __forceinline__ void warp_copy_realign(uint8_t* __restrict__ dst, const uint8_t* __restrict__ src,
                                                  int64_t n, int lane) {
  int64_t head = (int64_t)((0 - (uintptr_t)dst) & 15);
  if (head > n) head = n;
  const uint8_t hb = lane < head ? src[lane] : 0;
  const int64_t tail0 = (n - head) % 16;
  const uint8_t tb = lane < tail0 ? src[n - tail0 + lane] : 0;
  uint8_t* const dst0 = dst;
  dst += head;
  src += head;
  n -= head;
  const int64_t nv = n / 16;
  uint4* d = reinterpret_cast<uint4*>(dst);
  const uint4* A = reinterpret_cast<const uint4*>(src - R);  // (src - R) is 16-byte aligned
  constexpr int NWORD = (R + 15) / 4 - 3;  // words of the next vector that are needed (1..4)
  const int nb = (lane + 1) & 31;
  int64_t base = 0;
  for (; base + 32 * U <= nv; base += 32 * U) {
    uint4 a[U + 1];
#pragma unroll
    for (int u = 0; u < U; u++) a[u] = ldv<POL>(A + base + lane + 32 * u);
    a[U] = lane == 0 ? ldv<POL>(A + base + 32 * U) : make_uint4(0, 0, 0, 0);
    uint4 rot[U + 1];
#pragma unroll
    for (int u = 0; u <= U; u++) {
      rot[u].x = __shfl_sync(0xffffffffu, a[u].x, nb);
      if (NWORD > 1) rot[u].y = __shfl_sync(0xffffffffu, a[u].y, nb);
      if (NWORD > 2) rot[u].z = __shfl_sync(0xffffffffu, a[u].z, nb);
      if (NWORD > 3) rot[u].w = __shfl_sync(0xffffffffu, a[u].w, nb);
    }
#pragma unroll
    for (int u = 0; u < U; u++) {
      const uint4 nx = lane == 31 ? rot[u + 1] : rot[u];
      stv(d + base + lane + 32 * u, realign<R>(a[u], nx));
    }
  }
  for (int64_t i = base + lane; i < nv; i += 32 * U) {  // remainder (< 32*U vectors): one predicated batch
    uint4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; u++) {  // clamped (always valid) addresses keep the arrays in registers
      const int64_t j = min(i + 32 * u, nv - 1);
      a[u] = ldv<POL>(A + j);
      b[u] = ldv<POL>(A + j + 1);
    }
#pragma unroll
    for (int u = 0; u < U; u++)
      if (i + 32 * u < nv) stv(d + i + 32 * u, realign<R>(a[u], b[u]));
  }
  if (lane < head) dst0[lane] = hb;
  if (lane < tail0) dst[nv * 16 + lane] = tb;
}

template <int POL>
__device__ __forceinline__ void warp_copy(uint8_t* dst, const uint8_t* src, int64_t n, int lane) {
  if (n <= 0) return;
  const unsigned rel = (unsigned)(((uintptr_t)src - (uintptr_t)dst) & 15);
  // 4 KiB in flight per warp and iteration (memory-level parallelism: ~24-40
  // warps/SM x 4 KiB covers the loaded HBM latency).  Short segments take the
  // plain path (the realigning loop needs >= 32 vectors to pay off).
  if (rel == 0) { warp_copy_v<POL, uint4, 8>(dst, src, n, lane); return; }
  if (n < 1024) {
    if ((rel & 7) == 0) warp_copy_v<POL, uint2, 8>(dst, src, n, lane);
    else if ((rel & 3) == 0) warp_copy_v<POL, unsigned int, 8>(dst, src, n, lane);
    else warp_copy_v<POL, unsigned char, 8>(dst, src, n, lane);
    return;
  }
  switch (rel) {
    case 8: warp_copy_realign<POL, 8, 4>(dst, src, n, lane); break;
    case 4: warp_copy_realign<POL, 4, 4>(dst, src, n, lane); break;
    case 12: warp_copy_realign<POL, 12, 4>(dst, src, n, lane); break;
    case 1: warp_copy_realign<POL, 1, 4>(dst, src, n, lane); break;
    case 2: warp_copy_realign<POL, 2, 4>(dst, src, n, lane); break;
    case 3: warp_copy_realign<POL, 3, 4>(dst, src, n, lane); break;
    case 5: warp_copy_realign<POL, 5, 4>(dst, src, n, lane); break;
    case 6: warp_copy_realign<POL, 6, 4>(dst, src, n, lane); break;
    case 7: warp_copy_realign<POL, 7, 4>(dst, src, n, lane); break;
    case 9: warp_copy_realign<POL, 9, 4>(dst, src, n, lane); break;
    case 10: warp_copy_realign<POL, 10, 4>(dst, src, n, lane); break;
    case 11: warp_copy_realign<POL, 11, 4>(dst, src, n, lane); break;
    case 13: warp_copy_realign<POL, 13, 4>(dst, src, n, lane); break;
    case 14: warp_copy_realign<POL, 14, 4>(dst, src, n, lane); break;
    default: warp_copy_realign<POL, 15, 4>(dst, src, n, lane); break;
  }
}

// largest b with boff[b] <= q (boff strictly increasing, boff[0] == 0): 32-ary
// warp search, log32(nblocks) rounds of one coalesced probe each.
__device__ __forceinline__ int64_t warp_find_block(const int64_t* __restrict__ boff, int64_t nb, int64_t q,
                                                   int lane) {
  int64_t lo = 0, hi = nb;
  while (hi - lo > 1) {
    int64_t step = (hi - lo + 31) / 32;
    int64_t idx = lo + (int64_t)lane * step;
    bool ok = idx < hi && __ldg(boff + idx) <= q;
    unsigned m = __ballot_sync(0xffffffffu, ok);
    int k = 31 - __clz(m);  // lane 0 always true
    lo = lo + (int64_t)k * step;
    hi = min(hi, lo + step);
  }
  return lo;
}

// One warp copies stream bytes [p, p1) (P.pos <= p < p1 <= P.pos + P.len).
// POL applies to the loads (pack reads the layout, unpack reads the packed side).
// Walk from a resolved start: stream byte p is byte r of block b of element e
// (element displacement ed).  The next block's descriptor is prefetched while the
// current segment is copied.
// cb: packed-side base such that stream byte p lives at cb + p (cb = c - pos).
template <bool UNPACK, bool SINGLE, int POL>
__device__ __forceinline__ void seg_walk(const KP& P, uint8_t* cb, int64_t p, const int64_t p1, int64_t b, int64_t r,
                                         uint64_t e, int64_t ed, const int lane) {
  int64_t blen = SINGLE ? P.bl0 : __ldg(P.bl + b);
  int64_t bdsp = SINGLE ? P.bd0 : __ldg(P.bd + b);
  while (true) {
    const int64_t seg = min(blen - r, p1 - p);
    const int64_t nb = (SINGLE || b + 1 == P.nblocks) ? 0 : b + 1;
    int64_t nblen = 0, nbdsp = 0;
    if (!SINGLE && p + seg < p1) {
      nblen = __ldg(P.bl + nb);
      nbdsp = __ldg(P.bd + nb);
    }
    uint8_t* ncp = const_cast<uint8_t*>(P.nc) + ed + bdsp + r;
    uint8_t* cp = cb + p;
    if (UNPACK) warp_copy<POL>(ncp, cp, seg, lane);
    else warp_copy<POL>(cp, ncp, seg, lane);
    p += seg;
    if (p >= p1) break;
    r = 0;
    if (SINGLE || nb == 0) {
      ++e;
      ed = elem_disp(P, e);
    }
    b = nb;
    if (!SINGLE) {
      blen = nblen;
      bdsp = nbdsp;
    }
  }
}

template <bool UNPACK, bool SINGLE, int POL>
__device__ __forceinline__ void seg_range(const KP& P, uint8_t* cb, int64_t p, const int64_t p1, const int lane) {
  if (p >= p1) return;
  uint64_t e = fdiv((uint64_t)p, P.ftsize);
  int64_t r = p - (int64_t)e * P.tsize;
  int64_t b = 0;
  if (!SINGLE) {
    b = warp_find_block(P.boff, P.nblocks, r, lane);
    r -= __ldg(P.boff + b);
  }
  seg_walk<UNPACK, SINGLE, POL>(P, cb, p, p1, b, r, e, elem_disp(P, e), lane);
}

// ---------------------------------------------------------------- fused type -> type
// f1: stream bytes [p, p1) go from the source layout S straight to
// the destination layout R, no packed buffer.  Both sides keep a block cursor;
// each step copies min(rest of S's block, rest of R's block) with the relative
// alignment machinery of warp_copy.
struct Cursor {
  uint64_t e;
  int64_t b, r, ed, blen, bd;
};
__device__ __forceinline__ void cursor_init(const KP& P, Cursor& c, int64_t p, int lane) {
  c.e = fdiv((uint64_t)p, P.ftsize);
  c.r = p - (int64_t)c.e * P.tsize;
  c.b = 0;
  if (P.nblocks > 1) {
    c.b = warp_find_block(P.boff, P.nblocks, c.r, lane);
    c.r -= __ldg(P.boff + c.b);
  }
  c.ed = elem_disp(P, c.e);
  c.blen = P.nblocks == 1 ? P.bl0 : __ldg(P.bl + c.b);
  c.bd = P.nblocks == 1 ? P.bd0 : __ldg(P.bd + c.b);
}
__device__ __forceinline__ void cursor_advance(const KP& P, Cursor& c, int64_t n) {
  c.r += n;
  if (c.r < c.blen) return;
  c.r = 0;
  if (P.nblocks == 1 || ++c.b == P.nblocks) {
    c.b = 0;
    ++c.e;
    c.ed = elem_disp(P, c.e);
  }
  c.blen = P.nblocks == 1 ? P.bl0 : __ldg(P.bl + c.b);
  c.bd = P.nblocks == 1 ? P.bd0 : __ldg(P.bd + c.b);
}
__device__ __forceinline__ void dual_walk(const KP& S, const KP& R, int64_t p, const int64_t p1, int lane) {
  if (p >= p1) return;
  Cursor cs, cr;
  cursor_init(S, cs, p, lane);
  cursor_init(R, cr, p, lane);
  while (p < p1) {
    int64_t seg = min(cs.blen - cs.r, cr.blen - cr.r);
    seg = min(seg, p1 - p);
    const uint8_t* src = S.nc + cs.ed + cs.bd + cs.r;
    uint8_t* dst = const_cast<uint8_t*>(R.nc) + cr.ed + cr.bd + cr.r;
    warp_copy<LD_CS>(dst, src, seg, lane);
    p += seg;
    if (p >= p1) break;
    cursor_advance(S, cs, seg);
    cursor_advance(R, cr, seg);
  }
}

// ---------------------------------------------------------------- launch plans
// Cost-balanced warp slices (long-run kernel).  A warp's time is its bytes plus a
// fixed cost per segment (descriptor fetch + one memory round trip), so slices
// are cut at equal COST, cost(p) = p + alpha * (#block starts before p), instead
// of equal bytes: the triangle's tail of short columns is spread over many warps
// instead of serialising in the last one.  The cut positions depend only on the
// layout and (count, pos, len, nwarps), so they are computed once by k_plan and
// cached on the committed type — the paper's cached work distribution
// ([L18:c1649 §3.2]) without a per-unit array.
struct PlanEnt {
  int64_t p, b, r, e, ed;  // stream byte p = byte r of block b of element e (displacement ed)
};

// position of cost C (relative to cost 0 = stream byte 0), with its block/element
__device__ __forceinline__ PlanEnt pos_of_cost(const KP& P, int64_t alpha, const FastDiv& fce, int64_t ce, int64_t C) {
  const uint64_t e = fdiv((uint64_t)C, fce);
  const int64_t rc = C - (int64_t)e * ce;
  int64_t lo = 0, hi = P.nblocks;  // largest b with boff[b] + alpha*b <= rc
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) >> 1;
    if (__ldg(P.boff + mid) + alpha * mid <= rc) lo = mid;
    else hi = mid;
  }
  const int64_t off = rc - (__ldg(P.boff + lo) + alpha * lo);
  const int64_t bl = P.nblocks == 1 ? P.bl0 : __ldg(P.bl + lo);  // (a merged run lives in bl0)
  PlanEnt r;
  r.e = e;
  r.b = lo;
  r.r = min(off, bl);
  r.p = (int64_t)e * P.tsize + __ldg(P.boff + lo) + r.r;
  if (off >= bl) {  // inside the block's fixed cost: start at the next block
    r.r = 0;
    if (lo + 1 == P.nblocks) { r.b = 0; r.e = e + 1; }
    else r.b = lo + 1;
  }
  r.ed = 0;
  return r;
}

template <int G>
struct WordT;
template <> struct WordT<1> { typedef unsigned char T; };
template <> struct WordT<2> { typedef unsigned short T; };
template <> struct WordT<4> { typedef unsigned int T; };
template <> struct WordT<8> { typedef unsigned long long T; };
template <> struct WordT<16> { typedef uint4 T; };

// Threads tid, tid+nthr, ... each handle one VW-byte vector of the packed
// stream [lo, hi) (G-aligned, G-granular; cb + lo VW-aligned); wt is the
// template's word table in shared memory (nullptr for a single-block template).
// NV vectors per thread and iteration: every load of the batch is issued before
// the first store, so a thread keeps NV*VW bytes in flight.
template <bool UNPACK, int G, int VW, int POL, int NV = 2>
__device__ __forceinline__ void word_range(const KP& P, uint8_t* cb, const int64_t lo, const int64_t hi,
                                           const int32_t* wt, int64_t tid, int64_t nthr) {
  typedef typename WordT<G>::T W;
  typedef typename WordT<VW>::T VT;
  constexpr int NW = VW / G;
  const int64_t nvec = (hi - lo + VW - 1) / VW;
  const int64_t end = hi;
  uint8_t* const cv = cb + lo;  // vector v of the range lives at cv + v*VW
  union U {
    VT vec;
    W word[NW];
  };
  for (int64_t v0 = tid; v0 < nvec; v0 += nthr * NV) {
    U u[NV];
    int nvalid[NV];
    int64_t ed[NV], edn[NV];
    uint64_t e[NV];
    int w[NV];
    // when an element holds >= VW bytes a vector crosses at most one element
    // boundary: the next element's displacement (a list-table load for index
    // lists) is fetched up front instead of on the critical path mid-vector
    const bool one_cross = P.tsize >= VW;
#pragma unroll
    for (int j = 0; j < NV; j++) {
      const int64_t v = v0 + (int64_t)j * nthr;
      const int64_t s0 = lo + v * VW;
      const int64_t rem = v < nvec ? (end - s0) / G : 0;
      nvalid[j] = rem < NW ? (int)rem : NW;
      e[j] = fdiv((uint64_t)s0, P.ftsize);
      w[j] = (int)((s0 - (int64_t)e[j] * P.tsize) / G);
      ed[j] = nvalid[j] > 0 ? elem_disp(P, e[j]) : 0;
      edn[j] = (one_cross && nvalid[j] > 0 && w[j] + nvalid[j] > P.nwords) ? elem_disp(P, e[j] + 1) : 0;
      if (UNPACK) {
        if (nvalid[j] == NW) u[j].vec = ldv<POL>(reinterpret_cast<const VT*>(cv + v * VW));
        else
          for (int k = 0; k < nvalid[j]; k++) u[j].word[k] = reinterpret_cast<const W*>(cv + v * VW)[k];
      }
    }
#pragma unroll
    for (int j = 0; j < NV; j++) {
#pragma unroll
      for (int k = 0; k < NW; k++) {
        if (k < nvalid[j]) {
          // (wt == nullptr: single-block template, word k at bd0 + k*G -- no table load)
          const int64_t wo = wt ? (int64_t)wt[w[j]] : P.bd0 + (int64_t)w[j] * G;
          W* a = reinterpret_cast<W*>(const_cast<uint8_t*>(P.nc) + ed[j] + wo);
          if (UNPACK) *a = u[j].word[k];
          else u[j].word[k] = ldv<POL>(a);
          if (++w[j] == P.nwords && k + 1 < nvalid[j]) {
            w[j] = 0;
            ++e[j];
            ed[j] = one_cross ? edn[j] : elem_disp(P, e[j]);
          }
        }
      }
    }
    if (!UNPACK) {
#pragma unroll
      for (int j = 0; j < NV; j++) {
        const int64_t v = v0 + (int64_t)j * nthr;
        if (nvalid[j] == NW) stv(reinterpret_cast<VT*>(cv + v * VW), u[j].vec);
        else
          for (int k = 0; k < nvalid[j]; k++) reinterpret_cast<W*>(cv + v * VW)[k] = u[j].word[k];
      }
    }
  }
}

// ---------------------------------------------------------------- async staging
// cp.async (LDGSTS) gathers G-byte words straight into shared memory without
// holding them in registers, so a CTA keeps tens of KiB in flight; the
// contiguous side moves with TMA bulk copies (cp.async.bulk, UBLKCP): one
// instruction per tile.  This is the shared-memory/TMA staging of short runs.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int G>
__device__ __forceinline__ void cp_async(void* smem, const void* gmem) {
  if (G == 16)
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
  else
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(smem_u32(smem)), "l"(gmem), "n"(G) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_store(void* gmem, const void* smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gmem), "r"(smem_u32(smem)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_init(uint64_t* m, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_load(void* smem, const void* gmem, uint32_t bytes, uint64_t* m) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(smem)),
               "l"(gmem), "r"(bytes), "r"(smem_u32(m))
               : "memory");
}
// arrive (release at CTA scope: the arriving thread's prior writes precede a waiter's acquire)
__device__ __forceinline__ void mbar_arrive(uint64_t* m) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(m)) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t* m, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(smem_u32(m)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(m)),
      "r"(parity)
      : "memory");
}

constexpr int kStageTile = 16384;
constexpr int kStageBufs = 4;      // standalone kernels (several CTAs per SM)
constexpr int kXferStageBufs = 4;  // transfer kernel: per copy group (two groups per CTA)

// Element iterator: element e = hi*cnt[L] + lo over the innermost level L.  The
// displacement of the outer nest (hi) is cached; advancing by k elements touches
// only lo and recomputes the outer part when lo wraps (once per cnt[L] elements).
struct ElemIt {
  uint64_t hi;
  int64_t lo, hid;  // hid = displacement of element hi*cnt[L] without level L's contribution
  int L;
  __device__ __forceinline__ void init(const KP& P, uint64_t e) {
    L = P.nlev - 1;
    if (L < 0) { hi = e; lo = 0; hid = 0; return; }
    hi = fdiv(e, P.fcnt[L]);
    lo = (int64_t)(e - hi * (uint64_t)P.cnt[L]);
    outer(P);
  }
  __device__ __forceinline__ void outer(const KP& P) {
    const uint64_t e0 = hi * (uint64_t)P.cnt[L];
    hid = elem_disp(P, e0) - (P.table[L] ? __ldg(P.table[L]) : 0);
  }
  __device__ __forceinline__ int64_t disp(const KP& P) const {
    if (L < 0) return 0;
    return hid + (P.table[L] ? __ldg(P.table[L] + lo) : lo * P.stride[L]);
  }
  __device__ __forceinline__ void advance(const KP& P, int64_t k) {
    if (L < 0 || k == 0) return;
    lo += k;
    if (lo >= P.cnt[L]) {
      const uint64_t q = fdiv((uint64_t)lo, P.fcnt[L]);
      hi += q;
      lo -= (int64_t)q * P.cnt[L];
      outer(P);
    }
  }
};

// Word iterator: thread walks stream words x, x+S, x+2S, ... keeping (element,
// offset within the element) incrementally (one fast division per tile).
struct WordIt {
  uint64_t e;
  int64_t q, ed;
};

// Barrier over the threads that run a staged copy: the whole CTA (bar == 0) or one
// copy group of a warp-specialised kernel (named barrier `bar` over nthr threads).
__device__ __forceinline__ void group_sync(int bar, int nthr) {
  if (bar == 0) __syncthreads();
  else asm volatile("bar.sync %0, %1;" ::"r"(bar), "r"(nthr) : "memory");
}

// Pack stream bytes [lo, hi) (lo - P.pos and P.c 16-byte aligned) of a G-granular
// template through shared memory: per tile, every thread cp.async-gathers its
// words into the tile buffer; the finished tile leaves with one bulk store.
// NB tile buffers: NB-1 tiles of gathers in flight while the oldest finished tile
// is stored, so a CTA keeps (NB-1)*16 KiB of loads outstanding.
// PLAIN: the finished tile leaves with coalesced 16-byte stores of the group's threads
// instead of a TMA bulk store (a ring slot in another GPU's memory: generic-proxy
// stores over NVLink, ordered by the control warp's system-scope release)
template <int G, int NB, bool PLAIN = false>
__device__ __forceinline__ void stage_pack(const KP& P, uint8_t* cb, const int32_t* wt, int64_t lo, int64_t hi,
                                           uint8_t* sbuf, const int tid, const int nthr, const int bar = 0) {
  constexpr int T = kStageTile, L = NB - 1;
  const int64_t ntiles = (hi - lo + T - 1) / T;
  const int64_t S = (int64_t)nthr * G;  // a thread's stride through the stream: Se elements + Sq bytes
  const int64_t Se = (int64_t)fdiv((uint64_t)S, P.ftsize), Sq = S - Se * P.tsize;
  // Persistent per-thread word iterator: thread tid handles words tid, tid+nthr, ...
  // of the whole range (T/G is a multiple of nthr, so this is also its share of
  // every tile) -- one division and element decomposition per CALL, not per tile.
  const int64_t nwords = (hi - lo) / G;
  int64_t q = 0, ed = 0;
  ElemIt ei;
  if (tid < nwords) {
    const int64_t x0 = lo + (int64_t)tid * G;
    const uint64_t e0 = fdiv((uint64_t)x0, P.ftsize);
    q = x0 - (int64_t)e0 * P.tsize;
    ei.init(P, e0);
    ed = ei.disp(P);
  }
  int64_t iw = tid;  // next word of this thread (index from lo)
  for (int64_t t = 0; t < ntiles + L - 1; t++) {
    if (t < ntiles) {
      uint8_t* buf = sbuf + (t % NB) * T - (t * T);  // word iw lands at buf + iw*G
      if (!PLAIN && tid == 0) bulk_wait_read<1>();  // the store that last read this buffer (tile t-NB) is done reading
      group_sync(bar, nthr);
      const int64_t wend = (t + 1) * (T / G) < nwords ? (t + 1) * (T / G) : nwords;
      while (iw < wend) {
        cp_async<G>(buf + iw * G, P.nc + ed + wt[q / G]);
        iw += nthr;
        if (iw >= nwords) break;
        q += Sq;
        int64_t k = Se;
        if (q >= P.tsize) { q -= P.tsize; k++; }
        if (k) { ei.advance(P, k); ed = ei.disp(P); }
      }
    }
    cp_async_commit();  // (an empty group in the drain iterations keeps the group count uniform)
    const int64_t u = t - (L - 1);  // oldest tile in flight: store it once its gathers landed
    if (u >= 0) {
      cp_async_wait<L - 1>();
      group_sync(bar, nthr);
      if (PLAIN) {
        const int64_t s1 = lo + u * T;
        const int64_t tl = hi - s1 < T ? hi - s1 : (int64_t)T;
        const uint8_t* buf = sbuf + (u % NB) * T;
        const int nv = (int)(tl >> 4);
        for (int i = tid; i < nv; i += nthr)
          stv(reinterpret_cast<uint4*>(cb + s1) + i, reinterpret_cast<const uint4*>(buf)[i]);
        if (tid == 0)
          for (int64_t k = tl & ~int64_t(15); k < tl; k++) cb[s1 + k] = buf[k];  // ragged tail
      } else if (tid == 0) {
        const int64_t s1 = lo + u * T;
        const int64_t tl = hi - s1 < T ? hi - s1 : (int64_t)T;
        const uint8_t* buf = sbuf + (u % NB) * T;
        fence_proxy_async();
        if (tl >= 16) {
          bulk_store(cb + s1, buf, (uint32_t)(tl & ~int64_t(15)));
          bulk_commit();
        }
        for (int64_t k = tl & ~int64_t(15); k < tl; k++) cb[s1 + k] = buf[k];  // ragged tail
      }
    }
  }
  if (!PLAIN && tid == 0) bulk_wait_all();
}

// Unpack: tiles of the contiguous stream arrive by TMA bulk loads (NB in flight,
// mbarrier completion), then every thread scatters its words from shared memory.
// mbar[NB]: tb < 0 -- initialise them here (a standalone kernel, one call per CTA);
// tb >= 0 -- they were initialised once by the caller and tb tiles have gone through
// them before (a persistent kernel calling this per piece): tile t of this call uses
// buffer/mbarrier (tb + t) % NB at parity ((tb + t) / NB) & 1.  (Re-initialising an
// mbarrier per call makes ptxas invalidate the SYNCS unit's cached barrier state,
// which breaks another copy group's in-flight TMA transactions.)
template <int G, int NB>
__device__ __forceinline__ void stage_unpack(const KP& P, const uint8_t* cb, const int32_t* wt, int64_t lo, int64_t hi,
                                             uint8_t* sbuf, uint64_t* mbar, const int tid, const int nthr,
                                             const int bar = 0, int64_t tb = -1) {
  typedef typename WordT<G>::T W;
  constexpr int T = kStageTile;
  const int64_t ntiles = (hi - lo + T - 1) / T;
  const int64_t S = (int64_t)nthr * G;
  const int64_t Se = (int64_t)fdiv((uint64_t)S, P.ftsize), Sq = S - Se * P.tsize;
  if (tb < 0) {
    if (tid == 0) {
      for (int b = 0; b < NB; b++) mbar_init(mbar + b, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    group_sync(bar, nthr);
    tb = 0;
  }
  auto issue = [&](int64_t t) {
    const int64_t s = lo + t * T;
    const uint32_t bytes = (uint32_t)((hi - s < T ? hi - s : (int64_t)T) & ~int64_t(15));
    uint64_t* m = mbar + ((tb + t) % NB);
    mbar_expect_tx(m, bytes);
    if (bytes) bulk_load(sbuf + ((tb + t) % NB) * T, cb + s, bytes, m);
  };
  if (tid == 0)
    for (int64_t t = 0; t < NB && t < ntiles; t++) issue(t);
  // persistent per-thread word iterator (see stage_pack)
  const int64_t nwords = (hi - lo) / G;
  const int64_t fullw = ((hi - lo) & ~int64_t(15)) / G;  // words delivered through shared memory
  int64_t q = 0, ed = 0;
  ElemIt ei;
  if (tid < nwords) {
    const int64_t x0 = lo + (int64_t)tid * G;
    const uint64_t e0 = fdiv((uint64_t)x0, P.ftsize);
    q = x0 - (int64_t)e0 * P.tsize;
    ei.init(P, e0);
    ed = ei.disp(P);
  }
  int64_t iw = tid;
  for (int64_t t = 0; t < ntiles; t++) {
    const uint8_t* buf = sbuf + ((tb + t) % NB) * T - t * T;  // word iw of the range at buf + iw*G
    mbar_wait(mbar + ((tb + t) % NB), (uint32_t)(((tb + t) / NB) & 1));
    const int64_t wend = (t + 1) * (T / G) < nwords ? (t + 1) * (T / G) : nwords;
    while (iw < wend) {
      const W v = iw < fullw ? *reinterpret_cast<const W*>(buf + iw * G)
                             : *reinterpret_cast<const W*>(cb + lo + iw * G);  // ragged tail (< 16 B)
      *reinterpret_cast<W*>(const_cast<uint8_t*>(P.nc) + ed + wt[q / G]) = v;
      iw += nthr;
      if (iw >= nwords) break;
      q += Sq;
      int64_t k = Se;
      if (q >= P.tsize) { q -= P.tsize; k++; }
      if (k) { ei.advance(P, k); ed = ei.disp(P); }
    }
    group_sync(bar, nthr);  // buffer consumed
    if (tid == 0 && t + NB < ntiles) issue(t + NB);
  }
}

// Persistent word cursor of one layout: thread's words tid, tid+nthr, ... of [lo, ..)
struct WordCursor {
  int64_t q, ed, Se, Sq;
  ElemIt ei;
  __device__ __forceinline__ void init(const KP& P, int64_t x0, int64_t stride_bytes) {
    const uint64_t e0 = fdiv((uint64_t)x0, P.ftsize);
    q = x0 - (int64_t)e0 * P.tsize;
    ei.init(P, e0);
    ed = ei.disp(P);
    Se = (int64_t)fdiv((uint64_t)stride_bytes, P.ftsize);
    Sq = stride_bytes - Se * P.tsize;
  }
  __device__ __forceinline__ int64_t addr_off(const int32_t* wt, int G) const { return ed + wt[q / G]; }
  __device__ __forceinline__ void next(const KP& P) {
    q += Sq;
    int64_t k = Se;
    if (q >= P.tsize) { q -= P.tsize; k++; }
    if (k) { ei.advance(P, k); ed = ei.disp(P); }
  }
};

// Fused type -> type copy staged through shared memory: per 16 KiB tile of the
// stream, cp.async gathers the words from the source layout S (NB-1 tiles in
// flight), then the tile is scattered from shared memory to the destination
// layout R.  Each thread keeps a persistent cursor per layout.
template <int G, int NB>
__device__ __forceinline__ void stage_copy(const KP& S, const int32_t* wts, const KP& R, const int32_t* wtr,
                                           int64_t lo, int64_t hi, uint8_t* sbuf) {
  typedef typename WordT<G>::T W;
  constexpr int T = kStageTile, L = NB - 1;
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int64_t ntiles = (hi - lo + T - 1) / T;
  const int64_t nwords = (hi - lo) / G;
  WordCursor cs, cr;
  if (tid < nwords) {
    cs.init(S, lo + (int64_t)tid * G, (int64_t)nthr * G);
    cr.init(R, lo + (int64_t)tid * G, (int64_t)nthr * G);
  }
  int64_t iw = tid, jw = tid;
  for (int64_t t = 0; t < ntiles + L - 1; t++) {
    if (t < ntiles) {
      uint8_t* buf = sbuf + (t % NB) * T - t * T;
      const int64_t wend = (t + 1) * (T / G) < nwords ? (t + 1) * (T / G) : nwords;
      while (iw < wend) {
        cp_async<G>(buf + iw * G, S.nc + cs.addr_off(wts, G));
        iw += nthr;
        if (iw >= nwords) break;
        cs.next(S);
      }
    }
    cp_async_commit();
    const int64_t u = t - (L - 1);
    if (u >= 0) {
      cp_async_wait<L - 1>();
      __syncthreads();
      const uint8_t* buf = sbuf + (u % NB) * T - u * T;
      const int64_t wend = (u + 1) * (T / G) < nwords ? (u + 1) * (T / G) : nwords;
      while (jw < wend) {
        *reinterpret_cast<W*>(const_cast<uint8_t*>(R.nc) + cr.addr_off(wtr, G)) =
            *reinterpret_cast<const W*>(buf + jw * G);
        jw += nthr;
        if (jw >= nwords) break;
        cr.next(R);
      }
      __syncthreads();  // tile buffer free for the gather NB tiles later
    }
  }
}

// Fused type -> type copy of G-granular templates: thread tid moves words tid,
// tid+nthr, ... of [lo, hi): source address from S's word table + element
// iterator, destination from R's; NV words in flight per thread.
template <int G, int NV>
__device__ __forceinline__ void dual_words(const KP& S, const int32_t* wts, const KP& R, const int32_t* wtr,
                                           int64_t lo, int64_t hi, int64_t tid, int64_t nthr) {
  typedef typename WordT<G>::T W;
  const int64_t nwords = (hi - lo) / G;
  if (tid >= nwords) return;
  const int64_t St = nthr * G;
  const int64_t Ses = (int64_t)fdiv((uint64_t)St, S.ftsize), Sqs = St - Ses * S.tsize;
  const int64_t Ser = (int64_t)fdiv((uint64_t)St, R.ftsize), Sqr = St - Ser * R.tsize;
  const int64_t x0 = lo + tid * G;
  uint64_t e = fdiv((uint64_t)x0, S.ftsize);
  int64_t qs = x0 - (int64_t)e * S.tsize;
  ElemIt is;
  is.init(S, e);
  int64_t eds = is.disp(S);
  e = fdiv((uint64_t)x0, R.ftsize);
  int64_t qr = x0 - (int64_t)e * R.tsize;
  ElemIt ir;
  ir.init(R, e);
  int64_t edr = ir.disp(R);
  for (int64_t w = tid; w < nwords; w += nthr * NV) {
    W v[NV];
    W* d[NV];
#pragma unroll
    for (int j = 0; j < NV; j++) {
      if (w + j * nthr < nwords) {
        v[j] = ldv<LD_CS>(reinterpret_cast<const W*>(S.nc + eds + wts[qs / G]));
        d[j] = reinterpret_cast<W*>(const_cast<uint8_t*>(R.nc) + edr + wtr[qr / G]);
        if (w + (j + 1) * nthr >= nwords) continue;  // never step an iterator past the stream
        qs += Sqs;
        int64_t k = Ses;
        if (qs >= S.tsize) { qs -= S.tsize; k++; }
        if (k) { is.advance(S, k); eds = is.disp(S); }
        qr += Sqr;
        k = Ser;
        if (qr >= R.tsize) { qr -= R.tsize; k++; }
        if (k) { ir.advance(R, k); edr = ir.disp(R); }
      }
    }
#pragma unroll
    for (int j = 0; j < NV; j++)
      if (w + j * nthr < nwords) *d[j] = v[j];
  }
}

// Short blocks under a large template (irregular hindexed, C5b): a warp walks its
// stream slice in 512-byte windows.  For each window, lanes take one block each
// (32 per round, block starts from boff) and write the source address of every
// G-byte word their block contributes to the window into a per-warp shared
// table; then each lane moves its 16 output bytes: G-byte gathers from the
// table's addresses and one coalesced 16-byte store (unpack: the reverse).
constexpr int kBlkWin = 512;
template <bool UNPACK, int G, int POL>
__device__ __forceinline__ void blk_range(const KP& P, uint8_t* cbase, int64_t p0, const int64_t p1, int lane,
                                          int64_t* sa) {
  typedef typename WordT<G>::T W;
  const FastDiv& fnb = P.fnb;
  constexpr int NWL = 16 / G;  // words per lane
  if (p0 >= p1) return;
  uint64_t ce = fdiv((uint64_t)p0, P.ftsize);
  int64_t cb = warp_find_block(P.boff, P.nblocks, p0 - (int64_t)ce * P.tsize, lane);
  const uint64_t nel = P.nblocks ? (uint64_t)((p1 + P.tsize - 1) / P.tsize) : 0;  // elements this warp can touch
  for (int64_t q = p0; q < p1; q += kBlkWin) {
    const int64_t qe = min(q + kBlkWin, p1);
    while (true) {
      int64_t lb = cb + lane;
      uint64_t le = ce;
      if (lb >= P.nblocks) {
        const uint64_t k = fdiv((uint64_t)lb, fnb);
        le += k;
        lb -= (int64_t)k * P.nblocks;
      }
      int64_t start = INT64_MAX, len = 0;
      if (le < nel) {
        start = (int64_t)le * P.tsize + __ldg(P.boff + lb);
        len = __ldg(P.bl + lb);
      }
      const int64_t a = max(start, q), z = min(start + len, qe);
      if (a < z) {
        const int64_t base = (int64_t)(uintptr_t)P.nc + elem_disp(P, le) + __ldg(P.bd + lb) - start;
        for (int64_t x = a; x < z; x += G) sa[(x - q) / G] = base + x;
      }
      const bool reach = start != INT64_MAX && start + len >= qe;
      if (__any_sync(0xffffffffu, reach || start == INT64_MAX)) {
        const unsigned before = __ballot_sync(0xffffffffu, start != INT64_MAX && start + len <= qe);
        cb += __popc(before);
        break;
      }
      cb += 32;
    }
    if (cb >= P.nblocks) {
      const uint64_t k = fdiv((uint64_t)cb, fnb);
      ce += k;
      cb -= (int64_t)k * P.nblocks;
    }
    __syncwarp();
    const int64_t x0 = q + (int64_t)lane * 16;
    const int64_t remw = x0 >= qe ? 0 : (qe - x0) / G;
    const int nvalid = remw < NWL ? (int)remw : NWL;
    uint8_t* cp = cbase + x0;
    union {
      uint4 vec;
      W word[NWL];
    } u;
    if (UNPACK) {
      if (nvalid == NWL) u.vec = ldv<POL>(reinterpret_cast<const uint4*>(cp));
      else
        for (int k = 0; k < nvalid; k++) u.word[k] = reinterpret_cast<const W*>(cp)[k];
    }
#pragma unroll
    for (int k = 0; k < NWL; k++) {
      if (k < nvalid) {
        W* a = reinterpret_cast<W*>(sa[lane * NWL + k]);
        if (UNPACK) *a = u.word[k];
        else u.word[k] = ldv<POL>(a);
      }
    }
    if (!UNPACK) {
      if (nvalid == NWL) stv(reinterpret_cast<uint4*>(cp), u.vec);
      else
        for (int k = 0; k < nvalid; k++) reinterpret_cast<W*>(cp)[k] = u.word[k];
    }
    __syncwarp();
  }
}

// ---------------------------------------------------------------- block spans
// Short blocks of a large irregular block list (C5b: hindexed of 4..64-byte
// blocks with 0..60-byte gaps; too many blocks for a word table).  A warp takes
// the next 32 blocks of its slice as one window (lane i = block cb+i):
//   * the window's descriptors (len, disp) arrive by cp.async into shared memory;
//     its packed offsets are an inclusive warp-shuffle scan of the lengths (the
//     paper's prefix-sum offsets, [L16:c5201 §3.2]) -- no boff[] traffic after
//     the first block of the slice is found;
//   * the window's layout span [lo, hi) is one warp-wide min/max reduction;
//     when it fits kSpanBuf bytes the span moves as 16-byte chunks:
//     pack:   the span's 16-byte chunks land in shared memory, a
//             per-warp packed word map (span word of every packed word), then
//             each lane assembles whole 16-byte packed chunks (coalesced
//             stores; G-byte stores only at the window's two ends);
//     unpack: the packed window lands in shared memory, a per-warp span word map (packed
//             word of every covered span word), then each lane writes span
//             chunks in address order -- one 16-byte store when the window
//             covers the whole chunk, G-byte stores of the covered words
//             otherwise (bytes outside the typemap are never written);
//   * a wider span falls back to a warp-cooperative copy per block;
//   * two-stage software pipeline: while window k is copied, the loads of window
//     k+1 (its span or packed bytes: ONE TMA bulk copy, completion on an mbarrier)
//     and the descriptors of window k+2 are in flight, so each window costs its
//     copy work, not a DRAM round trip.
// Every DRAM sector of the layout is requested once by a 16-byte access instead
// of once per G-byte word (the per-word gathers of blk_range).
#ifndef DT_SPAN_BUF
#define DT_SPAN_BUF 4096
#endif
#ifndef DT_SPAN_MINB
#define DT_SPAN_MINB 2
#endif
// layout span bytes per window (multiple of 16).  (Measured: 3 KiB spans with three
// 256-thread CTAs per SM -- 80 registers, 128-184 bytes of spills -- made C5b 64 MiB
// pack / unpack 70.6 / 94.2 us vs 53-56 / 78 us with 4 KiB and two CTAs.)
constexpr int kSpanBuf = DT_SPAN_BUF;
constexpr int kSpanOut = 2048;  // packed bytes per window (multiple of 16)
constexpr int kSpanOutB = kSpanOut + 32;
constexpr int kSpanDesc = 32 * 16;  // one window's (len, disp) pairs
// per-warp shared memory: pack  = 2 spans + packed word map (G >= 4) + 2 descriptor sets;
//                         unpack = 2 packed windows + span word map (G >= 4) + 2 descriptor sets
// (+ 2 mbarriers, at the end)
constexpr int kSpanPackSmem = 2 * kSpanBuf + kSpanOutB / 2 + 2 * kSpanDesc + 16;
constexpr int kSpanUnpackSmem = 2 * kSpanOutB + (kSpanBuf / 4) * 2 + 2 * kSpanDesc + 16;
constexpr int kSpanWarpSmem = kSpanPackSmem > kSpanUnpackSmem ? kSpanPackSmem : kSpanUnpackSmem;

// Move `n` bytes (a multiple of G) between the packed stream at global `g` and
// shared memory at `s` with s == g (mod 16): G-byte head words up to 16-byte
// alignment, 16-byte vectors, G-byte tail words.  TO_SMEM: g -> s by cp.async
// (the caller commits and waits), else s -> g by stores.
template <bool TO_SMEM, int G, int POL>
__device__ __forceinline__ void span_window_io(uint8_t* g, uint8_t* s, int n, int lane) {
  typedef typename WordT<G>::T W;
  const int head = min(n, (int)((16 - ((uintptr_t)g & 15)) & 15));
  const int hw = head / G;
  if (lane < hw) {
    if (TO_SMEM && POL == LD_CG) reinterpret_cast<W*>(s)[lane] = __ldcg(reinterpret_cast<const W*>(g) + lane);
    else if (TO_SMEM) cp_async<G>(s + lane * G, g + lane * G);
    else reinterpret_cast<W*>(g)[lane] = reinterpret_cast<const W*>(s)[lane];
  }
  const int nv = (n - head) >> 4;
  uint4* gv = reinterpret_cast<uint4*>(g + head);
  uint4* sv = reinterpret_cast<uint4*>(s + head);
  for (int i = lane; i < nv; i += 32) {
    if (TO_SMEM) cp_async<16>(sv + i, gv + i);
    else stv(gv + i, sv[i]);
  }
  const int tw = (n - head - nv * 16) / G;
  if (lane < tw) {
    W* gt = reinterpret_cast<W*>(g + head + nv * 16);
    W* st = reinterpret_cast<W*>(s + head + nv * 16);
    if (TO_SMEM && POL == LD_CG) st[lane] = __ldcg(gt + lane);
    else if (TO_SMEM) cp_async<G>(st + lane, gt + lane);
    else gt[lane] = st[lane];
  }
}

// Wide span (scattered or unsorted blocks): blocks shorter than 256 bytes are
// copied by their own lane with G-byte words (the window's 32 blocks in flight at
// once), longer ones by the whole warp.  Not inlined, so that the realigning
// copies' registers do not cap the fast path.
template <bool UNPACK, int G, int POL>
__device__ __noinline__ void span_wide(int32_t n, int64_t a, int32_t off, uint8_t* cp, int lane) {
  typedef typename WordT<G>::T W;
  if (n > 0 && n < 256) {
    W* lw = reinterpret_cast<W*>(a);
    W* pw = reinterpret_cast<W*>(cp + off);
    const int nw = n / G;
#pragma unroll 4
    for (int i = 0; i < nw; i++) {
      if (UNPACK) lw[i] = POL == LD_CG ? __ldcg(pw + i) : pw[i];  // (ring slots: L2 only)
      else pw[i] = lw[i];
    }
  }
  unsigned big = __ballot_sync(0xffffffffu, n >= 256);
  while (big) {
    const int j = __ffs(big) - 1;
    big &= big - 1;
    const int32_t nj = __shfl_sync(0xffffffffu, n, j);
    uint8_t* aj = reinterpret_cast<uint8_t*>(__shfl_sync(0xffffffffu, a, j));
    uint8_t* pj = cp + __shfl_sync(0xffffffffu, off, j);
    if (UNPACK) warp_copy<POL>(aj, pj, nj, lane);
    else warp_copy<POL>(pj, aj, nj, lane);
  }
}

// m[at + i] = val + i for i < n, two entries per 4-byte store
__device__ __forceinline__ void map_fill(uint16_t* m, int at, int val, int n) {
  int i = 0;
  if ((at & 1) && n > 0) {
    m[at] = (uint16_t)val;
    i = 1;
  }
#pragma unroll 4
  for (; i + 1 < n; i += 2)
    *reinterpret_cast<uint32_t*>(m + at + i) = (uint32_t)(val + i) | ((uint32_t)(val + i + 1) << 16);
  if (i < n) m[at + i] = (uint16_t)(val + i);
}

// Block cursor of a warp: stream byte p is byte r of template block cb of element ce.
struct SpanCur {
  int64_t p, r, cb, ced;
  uint64_t ce;
};
// Issue the descriptor loads of the window starting at the cursor into dsc
// (lane i: block cb+i, wrapping into later elements); returns the lane's element.
__device__ __forceinline__ uint64_t span_desc_issue(const KP& P, const SpanCur& c, int64_t* dsc, int lane) {
  int64_t b = c.cb + lane;
  uint64_t e = c.ce;
  if (b >= P.nblocks) {
    const uint64_t k = fdiv((uint64_t)b, P.fnb);
    e += k;
    b -= (int64_t)k * P.nblocks;
  }
  if (P.nblocks == 1) {
    dsc[2 * lane] = P.bl0;
    dsc[2 * lane + 1] = P.bd0;
  } else if (P.sdesc) {  // compact: (len, disp - group base) + the 32-block group's base
    cp_async<8>(dsc + 2 * lane, P.sdesc + b);
    cp_async<8>(dsc + 2 * lane + 1, P.wbase + (b >> 5));
  } else {
    cp_async<8>(dsc + 2 * lane, P.bl + b);
    cp_async<8>(dsc + 2 * lane + 1, P.bd + b);
  }
  return e;
}
// a landed descriptor pair -> (len, disp)
__device__ __forceinline__ void span_desc_get(const KP& P, const int64_t* dsc, int lane, int64_t& len, int64_t& disp) {
  const int64_t x = dsc[2 * lane], y = dsc[2 * lane + 1];
  if (P.sdesc && P.nblocks != 1) {
    len = (int64_t)((uint64_t)x >> 32);
    disp = y + (int64_t)(int32_t)(uint32_t)x;
  } else {
    len = x;
    disp = y;
  }
}
// One window's geometry (per lane: its block's share).
struct SpanWin {
  int64_t a;       // layout address of the lane's first byte (n > 0)
  int64_t base16;  // layout span start, 16-byte aligned
  uint8_t* cp;     // packed address of the window's first byte
  int32_t off, n, L, nch;
  bool fast;
};
// Window at cursor c from the landed descriptors; advances c past it.
__device__ __forceinline__ SpanWin span_geom(const KP& P, SpanCur& c, uint64_t e, const int64_t* dsc,
                                             uint8_t* cbase, int64_t p1, int lane) {
  constexpr unsigned FULL = 0xffffffffu;
  constexpr int32_t kClamp = 1 << 30;
  SpanWin w;
  const int64_t skip = lane == 0 ? c.r : 0;
  int64_t dlen, ddisp;
  span_desc_get(P, dsc, lane, dlen, ddisp);
  // lengths clamped to 4 KiB for the 32-bit scan: a window never exceeds kSpanOut
  const int32_t len = (int32_t)min(dlen - skip, (int64_t)4096);
  int32_t inc = len;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int32_t t = __shfl_up_sync(FULL, inc, d);
    if (lane >= d) inc += t;
  }
  w.off = inc - len;
  w.L = (int32_t)min((int64_t)min(kSpanOut, __shfl_sync(FULL, inc, 31)), p1 - c.p);
  w.n = max(0, min(inc, w.L) - w.off);  // lanes with n > 0 are a prefix (lane 0 always)
  w.a = 0;
  if (w.n > 0) w.a = (int64_t)(uintptr_t)P.nc + (e == c.ce ? c.ced : elem_disp(P, e)) + ddisp + skip;
  const int64_t a0 = __shfl_sync(FULL, w.a, 0);
  const int32_t rel = (int32_t)max((int64_t)-kClamp, min((int64_t)kClamp, w.a - a0));
  int32_t rlo = w.n > 0 ? rel : INT32_MAX, rhi = w.n > 0 ? rel + w.n : INT32_MIN;
#pragma unroll
  for (int d = 16; d; d >>= 1) {
    rlo = min(rlo, __shfl_xor_sync(FULL, rlo, d));
    rhi = max(rhi, __shfl_xor_sync(FULL, rhi, d));
  }
  w.base16 = (a0 + rlo) & ~(int64_t)15;
  const int64_t span = a0 + rhi - w.base16;
  w.fast = span <= kSpanBuf;
  w.nch = w.fast ? (int32_t)((span + 15) >> 4) : 0;
  w.cp = cbase + c.p;
  // advance the cursor past the window's L bytes
  const int j = __popc(__ballot_sync(FULL, inc <= w.L));  // whole blocks consumed (a prefix of lanes)
  const int32_t offj = __shfl_sync(FULL, w.off, j & 31);
  c.p += w.L;
  if (j == 32) {
    c.cb += 32;
    c.r = 0;
  } else {
    c.r = (j == 0 ? c.r : 0) + (w.L - offj);
    c.cb += j;
  }
  if (c.cb >= P.nblocks) {
    const uint64_t k = fdiv((uint64_t)c.cb, P.fnb);
    c.ce += k;
    c.cb -= (int64_t)k * P.nblocks;
    // (past the slice's end the element may not exist: a list level has no entry for it)
    if (c.p < p1) c.ced = elem_disp(P, c.ce);
  }
  return w;
}

// start of a warp's slice at stream byte p (a 32-ary block search; the standalone
// kernel takes it from a cached plan instead)
__device__ __forceinline__ PlanEnt span_start(const KP& P, int64_t p, int lane) {
  PlanEnt s;
  s.p = p;
  s.e = (int64_t)fdiv((uint64_t)p, P.ftsize);
  s.r = p - s.e * P.tsize;
  s.b = 0;
  if (P.nblocks != 1) {
    s.b = warp_find_block(P.boff, P.nblocks, s.r, lane);
    s.r -= __ldg(P.boff + s.b);
  }
  s.ed = elem_disp(P, (uint64_t)s.e);
  return s;
}

// One warp moves stream bytes [start.p, p1) (multiples of G; start = block b, byte
// r, element e of the plan); sm = kSpanWarpSmem bytes of 16-byte-aligned shared
// memory owned by the warp.
template <bool UNPACK, int G, int POL>
__device__ __forceinline__ void span_range(const KP& P, uint8_t* cbase, const PlanEnt& start, const int64_t p1,
                                           int lane, uint8_t* sm) {
  typedef typename WordT<G>::T W;
  constexpr int NWL = 16 / G;
  if (start.p >= p1) return;
  // shared-memory carve-up (see kSpanPackSmem / kSpanUnpackSmem)
  uint8_t* buf0 = sm;  // pack: span 0 | unpack: packed window 0
  uint8_t* buf1 = sm + (UNPACK ? kSpanOutB : kSpanBuf);
  uint16_t* omap = reinterpret_cast<uint16_t*>(sm + 2 * kSpanBuf);  // pack: packed word map
  uint16_t* wmap = reinterpret_cast<uint16_t*>(sm + 2 * kSpanOutB);  // unpack: span word map
  int64_t* dsc0 =
      reinterpret_cast<int64_t*>(sm + (UNPACK ? 2 * kSpanOutB + (kSpanBuf / 4) * 2 : 2 * kSpanBuf + kSpanOutB / 2));
  int64_t* dsc1 = dsc0 + 64;
  uint64_t* mb = reinterpret_cast<uint64_t*>(sm + kSpanWarpSmem - 16);  // one per span/window buffer
  if (lane == 0) {
    mbar_init(mb, 1);
    mbar_init(mb + 1, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  uint32_t phase = 0;  // bit s: parity of the next completion of buffer s
  SpanCur c;  // the warp's start, resolved by k_plan
  c.p = start.p;
  c.ce = (uint64_t)start.e;
  c.r = start.r;
  c.cb = start.b;
  c.ced = start.ed;
  // prologue: window 0's descriptors, geometry, loads; window 1's descriptors
  uint64_t e = span_desc_issue(P, c, dsc0, lane);
  cp_async_commit();
  cp_async_wait<0>();
  __syncwarp();
  SpanWin w = span_geom(P, c, e, dsc0, cbase, p1, lane);
  // one TMA bulk copy (UBLKCP) per window: the layout span (pack) or the 16-byte-aligned
  // hull of the packed window (unpack; buffer + (cp & 15) == cp mod 16), completion on mb[st]
  auto issue = [&](const SpanWin& x, uint8_t* b, int st) {
    if (!x.fast || lane != 0) return;
    const uint8_t* src;
    uint32_t bytes;
    if (UNPACK) {
      src = reinterpret_cast<const uint8_t*>((uintptr_t)x.cp & ~(uintptr_t)15);
      bytes = (uint32_t)((((uintptr_t)x.cp & 15) + x.L + 15) & ~15);
    } else {
      src = reinterpret_cast<const uint8_t*>(x.base16);
      bytes = (uint32_t)x.nch * 16u;
    }
    mbar_expect_tx(mb + st, bytes);
    bulk_load(b, src, bytes, mb + st);
  };
  issue(w, buf0, 0);
  if (c.p < p1) e = span_desc_issue(P, c, dsc1, lane);
  cp_async_commit();
  int k = 0;
  while (true) {
    cp_async_wait<0>();  // window k+1's descriptors have landed
    if (w.fast) {        // window k's bytes
      mbar_wait(mb + (k & 1), (phase >> (k & 1)) & 1u);
      phase ^= 1u << (k & 1);
    }
    __syncwarp();
    uint8_t* bk = (k & 1) ? buf1 : buf0;
    const bool more = c.p < p1;
    SpanWin nx;
    if (more) {
      int64_t* dn = (k & 1) ? dsc0 : dsc1;  // window k+1's descriptors
      nx = span_geom(P, c, e, dn, cbase, p1, lane);
      issue(nx, (k & 1) ? buf0 : buf1, (k + 1) & 1);
      if (c.p < p1) e = span_desc_issue(P, c, (k & 1) ? dsc1 : dsc0, lane);  // window k+2's
      cp_async_commit();
    }
    // ---- copy window k
    if (!w.fast) {
      span_wide<UNPACK, G, POL>(w.n, w.a, w.off, w.cp, lane);
    } else if (!UNPACK) {
      // packed-word map: omap[word of the window's 16-byte-aligned packed range] =
      // span word; then each lane assembles whole 16-byte packed chunks
      const int ob = (int)((uintptr_t)w.cp & 15);
      const int sw = (int)((w.a - w.base16) / G), ow = (ob + w.off) / G, nw = w.n / G;
      map_fill(omap, ow, sw, nw);
      __syncwarp();
      const W* sp = reinterpret_cast<const W*>(bk);
      const int w0 = ob / G, w1 = (ob + w.L) / G, nco = (ob + w.L + 15) >> 4;
      uint8_t* c16 = reinterpret_cast<uint8_t*>((uintptr_t)w.cp & ~(uintptr_t)15);
      for (int ch = lane; ch < nco; ch += 32) {
        union {
          uint16_t e[NWL];
          typename WordT<2 * NWL>::T all;
        } m;
        m.all = reinterpret_cast<const typename WordT<2 * NWL>::T*>(omap)[ch];
        union {
          uint4 v;
          W w[NWL];
        } u;
        const int wi = ch * NWL;
        if (wi >= w0 && wi + NWL <= w1) {
#pragma unroll
          for (int i = 0; i < NWL; i++) u.w[i] = sp[m.e[i]];
          stv(reinterpret_cast<uint4*>(c16 + 16 * ch), u.v);
        } else {
#pragma unroll
          for (int i = 0; i < NWL; i++)
            if (wi + i >= w0 && wi + i < w1) reinterpret_cast<W*>(c16 + 16 * ch)[i] = sp[m.e[i]];
        }
      }
      __syncwarp();
    } else {
      const int ob = (int)((uintptr_t)w.cp & 15);
      uint4* m4 = reinterpret_cast<uint4*>(wmap);  // 8 entries per 16-byte store
      for (int i = lane; i < (w.nch * NWL + 7) / 8; i += 32) m4[i] = make_uint4(~0u, ~0u, ~0u, ~0u);
      __syncwarp();
      const int sw = (int)((w.a - w.base16) / G), ow = (ob + w.off) / G, nw = w.n / G;
      map_fill(wmap, sw, ow, nw);
      __syncwarp();
      const W* owp = reinterpret_cast<const W*>(bk);
      for (int ch = lane; ch < w.nch; ch += 32) {
        union {
          uint16_t e[NWL];
          typename WordT<2 * NWL>::T all;
        } m;
        m.all = reinterpret_cast<const typename WordT<2 * NWL>::T*>(wmap)[ch];
        bool full = true;
#pragma unroll
        for (int i = 0; i < NWL; i++) full = full && m.e[i] != 0xFFFFu;
        uint8_t* d = reinterpret_cast<uint8_t*>(w.base16 + 16 * ch);
        if (full) {
          union {
            uint4 v;
            W w[NWL];
          } u;
#pragma unroll
          for (int i = 0; i < NWL; i++) u.w[i] = owp[m.e[i]];
          stv(reinterpret_cast<uint4*>(d), u.v);
        } else {
#pragma unroll
          for (int i = 0; i < NWL; i++)
            if (m.e[i] != 0xFFFFu) reinterpret_cast<W*>(d)[i] = owp[m.e[i]];
        }
      }
      __syncwarp();
    }
    if (!more) break;
    w = nx;
    k++;
  }
  // the warp's smem may be re-carved by its next call (next ring fragment): retire the
  // mbarriers (an mbarrier must be invalidated before its memory is re-initialised)
  __syncwarp();
  if (lane == 0) {
    asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(mb)) : "memory");
    asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(mb + 1)) : "memory");
  }
  __syncwarp();
}

// ---------------------------------------------------------------- record spans
// Short blocks inside small dense records (C5's 56-of-64-byte particles; any
// template whose blocks lie in a 16-byte-aligned span of <= 128 B that is at least
// half payload, with 16-byte-aligned element bases).  A warp moves RB whole
// records per batch (RB a multiple of 32, so every batch starts on a 16-byte
// boundary of the packed stream).
//   pack:   each lane issues its LPL 16-byte loads of the records' spans (all in
//           flight together; 4 lanes per 64-byte record), parks them in a per-warp
//           shared buffer, then assembles coalesced 16-byte vectors of the packed
//           stream from the template words (offset table `omap` in shared memory);
//   unpack: the packed vectors land in the shared buffer, each lane writes span
//           chunks: one 16-byte store when the template covers the chunk, G-byte
//           stores of the covered words otherwise (gap bytes stay untouched).
// Compared with gathering G-byte words (k_word), every DRAM sector of a record is
// requested by one 16-byte access instead of 16/G word accesses.
struct RecGeo {
  int64_t a0;          // span start relative to the element displacement (16-aligned)
  int32_t spanB, nch;  // span bytes (multiple of 16, <= 128) and 16-byte chunks
  int32_t RB, LPL;     // records per warp batch (multiple of 32), chunks per lane (RB*nch/32)
  int32_t nwr;         // template words per record (tsize / G)
  int32_t invnch;      // ceil(2^16 / nch): idx / nch = (idx * invnch) >> 16 for idx < 4096
  int64_t e_lo, e_hi;  // elements touching [pos, pos+len)
  int64_t b0, nbatch;  // first batch element (multiple of 32) and number of batches
  uint8_t woff[32];    // span word (G bytes) of packed word k of a record: in the kernel
                       // parameters, so no table load precedes the first gather
};
constexpr int kRecMaxLPL = 8;

// [lo, hi): the stream bytes this call may write (the request, or one pipeline fragment)
template <int G, int POL = LD_CS>
__device__ __forceinline__ void rec_pack_batch(const KP& P, const RecGeo& R, uint8_t* cb, int64_t e0, uint8_t* buf,
                                               const int64_t* sd, const uint16_t* omap, int lane, int64_t lo,
                                               int64_t end) {
  typedef typename WordT<G>::T W;
  constexpr int NW = 16 / G;
  uint4 v[kRecMaxLPL];
#pragma unroll
  for (int j = 0; j < kRecMaxLPL; j++) {
    if (j < R.LPL) {
      const int idx = lane + 32 * j;
      const int r = (idx * R.invnch) >> 16, ch = idx - r * R.nch;
      const int64_t e = e0 + r;
      if (e >= R.e_lo && e < R.e_hi) v[j] = ldv<POL>(reinterpret_cast<const uint4*>(P.nc + sd[r] + R.a0 + 16 * ch));
    }
  }
#pragma unroll
  for (int j = 0; j < kRecMaxLPL; j++)
    if (j < R.LPL) reinterpret_cast<uint4*>(buf)[lane + 32 * j] = v[j];  // (unloaded chunks: never output)
  __syncwarp();
  const int nvec = (int)((int64_t)R.RB * P.tsize / 16);  // RB is a multiple of 32: exact
  const int64_t sb = e0 * P.tsize;
  for (int vv = lane; vv < nvec; vv += 32) {
    const int64_t s = sb + 16 * (int64_t)vv;
    if (s + 16 <= lo || s >= end) continue;
    union {
      uint4 q;
      W w[NW];
    } o;
#pragma unroll
    for (int k = 0; k < NW; k++) o.w[k] = *reinterpret_cast<const W*>(buf + omap[vv * NW + k]);
    if (s >= lo && s + 16 <= end) {
      stv(reinterpret_cast<uint4*>(cb + s), o.q);
    } else {
      const uint8_t* ob = reinterpret_cast<const uint8_t*>(&o.q);
      for (int k = 0; k < 16; k++)
        if (s + k >= lo && s + k < end) cb[s + k] = ob[k];
    }
  }
  __syncwarp();
}

template <int G, int POL = LD_CS>
__device__ __forceinline__ void rec_unpack_batch(const KP& P, const RecGeo& R, const uint8_t* cb, int64_t e0,
                                                 uint8_t* buf, const int64_t* sd, const int16_t* umap, int lane,
                                                 int64_t lo, int64_t end) {
  typedef typename WordT<G>::T W;
  constexpr int NW = 16 / G;
  const int nvec = (int)((int64_t)R.RB * P.tsize / 16);
  const int64_t sb = e0 * P.tsize;
  uint4 v[kRecMaxLPL];
#pragma unroll
  for (int j = 0; j < kRecMaxLPL; j++) {  // nvec <= RB*spanB/16 = 32*LPL
    const int vv = lane + 32 * j;
    const int64_t s = sb + 16 * (int64_t)vv;
    if (j < R.LPL && vv < nvec && s >= lo && s + 16 <= end) v[j] = ldv<POL>(reinterpret_cast<const uint4*>(cb + s));
  }
#pragma unroll
  for (int j = 0; j < kRecMaxLPL; j++) {
    const int vv = lane + 32 * j;
    const int64_t s = sb + 16 * (int64_t)vv;
    if (j < R.LPL && vv < nvec) {
      if (s >= lo && s + 16 <= end) reinterpret_cast<uint4*>(buf)[vv] = v[j];
      else if (s + 16 > lo && s < end)  // ragged ends of the request: in-range words only
        for (int k = 0; k < 16; k += G)
          if (s + k >= lo && s + k + G <= end)
            *reinterpret_cast<W*>(buf + 16 * vv + k) = *reinterpret_cast<const W*>(cb + s + k);
    }
  }
  __syncwarp();
#pragma unroll
  for (int j = 0; j < kRecMaxLPL; j++) {
    if (j < R.LPL) {
      const int idx = lane + 32 * j;
      const int r = (idx * R.invnch) >> 16, ch = idx - r * R.nch;
      const int64_t e = e0 + r;
      if (e >= R.e_lo && e < R.e_hi) {
        const int64_t rs = e * P.tsize;  // stream byte of the record's first word
        const bool whole = rs >= lo && rs + P.tsize <= end;
        union {
          uint4 q;
          W w[NW];
        } o;
        unsigned mask = 0;
#pragma unroll
        for (int k = 0; k < NW; k++) {
          const int m = umap[ch * NW + k];
          if (m >= 0) {
            const int64_t x = rs + (int64_t)m * G;
            if (whole || (x >= lo && x + G <= end)) {
              o.w[k] = *reinterpret_cast<const W*>(buf + (int64_t)r * P.tsize + (int64_t)m * G);
              mask |= 1u << k;
            }
          }
        }
        uint8_t* d = const_cast<uint8_t*>(P.nc) + sd[r] + R.a0 + 16 * ch;
        if (mask == (1u << NW) - 1) {
          stv(reinterpret_cast<uint4*>(d), o.q);
        } else {
#pragma unroll
          for (int k = 0; k < NW; k++)
            if (mask & (1u << k)) reinterpret_cast<W*>(d)[k] = o.w[k];
        }
      }
    }
  }
  __syncwarp();
}

// Per-CTA maps of the record-span kernels from the span words of the template:
// pack -> omap[i] (tile word i -> shared byte), unpack -> umap[span word] (-1 = gap).
template <bool UNPACK, int G>
__device__ __forceinline__ void rec_maps(const RecGeo& R, uint16_t* omap) {
  if (!UNPACK) {
    const int n = R.RB * R.nwr;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      const int r = i / R.nwr, k = i - r * R.nwr;
      omap[i] = (uint16_t)(r * R.spanB + G * (int)R.woff[k]);
    }
  } else {
    int16_t* umap = reinterpret_cast<int16_t*>(omap);
    for (int i = threadIdx.x; i < R.spanB / G; i += blockDim.x) umap[i] = -1;
    __syncthreads();
    for (int k = threadIdx.x; k < R.nwr; k += blockDim.x) umap[R.woff[k]] = (int16_t)k;
  }
}

// Records of stream bytes [lo, hi) by the warps (w, nwt) of a grid: batch b of RB records
// starts at element R.b0 + b*RB (R.e_lo/e_hi/b0/nbatch describe [lo, hi)).
template <bool UNPACK, int G, int POL>
__device__ __forceinline__ void rec_range(const KP& P, const RecGeo& R, uint8_t* cb, int64_t lo, int64_t hi,
                                          uint8_t* buf, int64_t* sd, uint16_t* omap, int64_t w, int64_t nwt,
                                          int lane) {
  for (int64_t b = w; b < R.nbatch; b += nwt) {
    const int64_t e0 = R.b0 + b * R.RB;
    for (int i = lane; i < R.RB; i += 32) {
      const int64_t e = e0 + i;
      sd[i] = (e >= R.e_lo && e < R.e_hi) ? elem_disp(P, (uint64_t)e) : 0;
    }
    __syncwarp();
    if (UNPACK) rec_unpack_batch<G, POL>(P, R, cb, e0, buf, sd, reinterpret_cast<const int16_t*>(omap), lane, lo, hi);
    else rec_pack_batch<G, POL>(P, R, cb, e0, buf, sd, omap, lane, lo, hi);
  }
}

// ---------------------------------------------------------------- system-scope flags
// (cross-GPU signalling over NVLink peer memory: transfer rings and direct plans)
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_release_sys_add(uint64_t* p, uint64_t v) {
  asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// scope-selected flag operations: .gpu when both sides of a flag run on this GPU
// (loopback, two processes sharing a device), .sys across GPUs (NVLink peers)
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t* p, bool sys) {
  uint64_t v;
  if (sys) asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  else asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint64_t* p, uint64_t v, bool sys) {
  if (sys) asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t v, bool sys) {
  if (sys) asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

enum { XERR_TIMEOUT = 1, XERR_TRUNCATE = 2 };

// spin until pred(*p) holds; false on timeout (sets *err)
template <typename Pred>
__device__ __forceinline__ bool spin(const uint64_t* p, Pred pred, int64_t timeout_ns, int32_t* err, uint64_t* out,
                                     bool sleep = true, bool sys = true) {
  uint64_t v = ld_acquire(p, sys);
  if (pred(v)) { *out = v; return true; }
  const uint64_t t0 = gtimer();
  int ns = 32;
  while (true) {
    if (sleep) __nanosleep(ns);
    if (ns < 256) ns <<= 1;
    v = ld_acquire(p, sys);
    if (pred(v)) { *out = v; return true; }
    if ((int64_t)(gtimer() - t0) > timeout_ns) {
      atomicCAS(err, 0, XERR_TIMEOUT);
      return false;
    }
  }
}

// ---------------------------------------------------------------- host helpers (dt_kernels.cu)
dt_status dual_params(dt_type_s* st, int64_t scount, const void* src, dt_type_s* rt, int64_t rcount, void* dst,
                      int64_t n, KP& S, KP& R, int* kind, int64_t* gran);
int nonoverlap_cached(dt_type_s* rt, int64_t rcount);
bool rec_geometry(const Form& f, const KLevels& L, uint64_t nc_addr, uint64_t c_addr, int64_t pos, int64_t len,
                  int64_t g, RecGeo* R);

}  // namespace dt
