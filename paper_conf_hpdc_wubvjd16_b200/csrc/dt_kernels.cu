// dt_kernels.cu — sm_100a kernels of libdt and the pack/unpack entry points.
//
//   k_scan_*   device exclusive prefix of the template block lengths with warp
//              shuffles (the paper computes DEV packed displacements on the CPU,
//              [L16:c5996 §3.2]; here the scan runs on the GPU at commit).
//   k_seg      "warp-per-block" pack/unpack for long runs: every warp owns an
//              equal slice of the packed stream (the paper's equal-size CUDA DEVs
//              per warp, S = 1/2/4 KB, [L16:c5678]-[L18:c753 §3.2], so skewed block
//              lengths — the triangle — no longer cost occupancy, [L24:c282 §5.1]),
//              resolves its start position once (mixed-radix element index +
//              32-ary warp search over the block prefix) and walks block segments,
//              copying each with coalesced 16-byte vectors and head/tail peeling
//              ([L16:c2741]-[L16:c3777 §3.1]; the paper used 8 B/thread on Kepler).
//   k_word     "thread-per-element" pack/unpack for short blocks (4-64 B): a word
//              table of the template (granularity G) lives in shared memory, each
//              thread assembles one 16-byte vector of the packed stream, so the
//              contiguous side is written/read with full coalesced 16 B accesses.
//
// Everything is byte movement on integer vector types: no floating point.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <initializer_list>
#include <thread>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <climits>

#include "dt_device.cuh"
#include "dt_internal.h"

namespace dt {

// --------------------------------------------------------------- scan (K6)
// Block-wide exclusive scan of one int64 per thread using warp shuffles.
template <int NT>
__device__ __forceinline__ int64_t block_exclusive_scan(int64_t v, int64_t* total) {
  __shared__ int64_t wsum[NT / 32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int64_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int64_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[w] = x;
  __syncthreads();
  if (w == 0) {
    int64_t s = lane < NT / 32 ? wsum[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int64_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < NT / 32) wsum[lane] = s;  // inclusive warp prefix
  }
  __syncthreads();
  int64_t before = w ? wsum[w - 1] : 0;
  *total = wsum[NT / 32 - 1];
  __syncthreads();
  return before + x - v;
}

constexpr int kScanNT = 256, kScanItems = 4, kScanTile = kScanNT * kScanItems;

__global__ void __launch_bounds__(kScanNT) k_scan_local(const int64_t* __restrict__ in, int64_t* __restrict__ out,
                                                        int64_t* __restrict__ sums, int64_t n) {
  int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
  int64_t v[kScanItems], s = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; k++) {
    v[k] = base + k < n ? in[base + k] : 0;
    s += v[k];
  }
  int64_t tot;
  int64_t ex = block_exclusive_scan<kScanNT>(s, &tot);
#pragma unroll
  for (int k = 0; k < kScanItems; k++) {
    if (base + k < n) out[base + k] = ex;
    ex += v[k];
  }
  if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kScanNT) k_scan_sums(int64_t* sums, int64_t nb, int64_t carry0 = 0) {
  int64_t carry = carry0;
  for (int64_t b0 = 0; b0 < nb; b0 += kScanNT) {
    int64_t i = b0 + threadIdx.x;
    int64_t v = i < nb ? sums[i] : 0, tot;
    int64_t ex = block_exclusive_scan<kScanNT>(v, &tot);
    if (i < nb) sums[i] = carry + ex;
    carry += tot;
  }
}

__global__ void __launch_bounds__(kScanNT) k_scan_add(int64_t* out, const int64_t* sums, int64_t n) {
  int64_t base = (int64_t)blockIdx.x * kScanTile;
  int64_t add = sums[blockIdx.x];
  for (int k = threadIdx.x; k < kScanTile; k += kScanNT)
    if (base + k < n) out[base + k] += add;
}

// --------------------------------------------------------------- standalone kernels
// warp w of the long-run kernel copies stream bytes [plan[w].p, plan[w+1].p)
template <bool UNPACK, bool SINGLE>
__global__ void __launch_bounds__(256, 3) k_seg(const KP P, const PlanEnt* __restrict__ plan, int64_t nw) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= nw) return;
  const PlanEnt a = plan[gw];
  const int64_t p1 = plan[gw + 1].p;
  if (a.p >= p1) return;
  seg_walk<UNPACK, SINGLE, LD_CS>(P, P.c - P.pos, a.p, p1, a.b, a.r, a.e, a.ed, lane);
}

// single-block templates (every block the same length, so cost balance is moot):
// warp w copies [pos + w*per, ...) resolved arithmetically -- no plan load ahead
// of the first data load (latency-bound small messages: C1, C4 y/z faces)
template <bool UNPACK>
__global__ void __launch_bounds__(256, 3) k_seg_eq(const KP P, int64_t per) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t p = P.pos + gw * per, end = P.pos + P.len;
  if (p >= end) return;
  seg_range<UNPACK, true, LD_CS>(P, P.c - P.pos, p, min(p + per, end), lane);
}

// One contiguous 16-byte-aligned run (a contiguous layout, or a vector whose blocks abut):
// a grid-stride copy, 4 x 16 B per thread and iteration, many short CTAs.  At 2 GiB it
// reaches 0.965 of the same-run torch copy where k_seg_eq's one wave of equal per-warp
// slices reaches 0.90: neighbouring warps touch neighbouring bytes at the same time.
__global__ void __launch_bounds__(128) k_run_copy(const uint4* __restrict__ a, uint4* __restrict__ b, int64_t nv) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * 4;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x) * 4 + threadIdx.x; i < nv; i += stride) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; u++)
      if (i + u * 128 < nv) v[u] = __ldcs(a + i + u * 128);
#pragma unroll
    for (int u = 0; u < 4; u++)
      if (i + u * 128 < nv) __stcs(b + i + u * 128, v[u]);
  }
}

// one thread per warp boundary: cost-balanced cut positions (see PlanEnt)
// (gran > 1: cuts rounded down to multiples of gran bytes -- the block-span kernel
// moves whole G-byte words)
__global__ void k_plan(const KP P, int64_t alpha, FastDiv fce, int64_t ce, int64_t C0, int64_t C1, int64_t nw,
                       int64_t gran, PlanEnt* plan) {
  const int64_t w = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (w > nw) return;
  const int64_t C = w == nw ? C1 : C0 + (int64_t)((__int128)(C1 - C0) * w / nw);
  PlanEnt r = pos_of_cost(P, alpha, fce, ce, C);
  if (gran > 1) {
    const int64_t d = r.r % gran;
    r.r -= d;
    r.p -= d;
  }
  const int64_t end = P.pos + P.len;
  if (w == nw || r.p > end) r.p = end;
  if (r.p < P.pos) r.p = P.pos;
  r.ed = r.p < end ? elem_disp(P, r.e) : 0;
  plan[w] = r;
}

template <bool UNPACK, int G>
__global__ void __launch_bounds__(256) k_blk(const KP P) {
  extern __shared__ int64_t sa_all[];
  const int lane = threadIdx.x & 31;
  int64_t* sa = sa_all + (threadIdx.x >> 5) * (kBlkWin / G);
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t p = P.pos + gw * P.per_warp;
  const int64_t p1 = min(p + P.per_warp, P.pos + P.len);
  blk_range<UNPACK, G, LD_CS>(P, P.c - P.pos, p, p1, lane, sa);
}

// block-span pack/unpack (short blocks of a large irregular list): warp w owns
// stream bytes [pos + w*per_warp, ...) and walks them 32 blocks at a time
template <bool UNPACK, int G>
__global__ void __launch_bounds__(256, DT_SPAN_MINB) k_span(const KP P, const PlanEnt* __restrict__ plan, int64_t nw) {
  extern __shared__ __align__(16) uint8_t smem_span[];
  const int lane = threadIdx.x & 31;
  uint8_t* sm = smem_span + (threadIdx.x >> 5) * kSpanWarpSmem;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= nw) return;
  const PlanEnt a = plan[gw];
  span_range<UNPACK, G, LD_CS>(P, P.c - P.pos, a, plan[gw + 1].p, lane, sm);
}

// shared-memory staged pack/unpack (cp.async gathers / TMA bulk), CTA c owns a
// contiguous run of 16 KiB tiles of the stream
template <bool UNPACK, int G>
__global__ void __launch_bounds__(256) k_stage(const KP P, int64_t ntiles) {
  extern __shared__ __align__(128) uint8_t smem_stage[];
  __shared__ uint64_t mbar[kStageBufs];
  uint8_t* sbuf = smem_stage;
  int32_t* wt = reinterpret_cast<int32_t*>(smem_stage + kStageBufs * kStageTile);
  for (int i = threadIdx.x; i < P.nwords; i += blockDim.x) wt[i] = P.wtab[i];
  __syncthreads();
  const int64_t t0 = ntiles * blockIdx.x / gridDim.x, t1 = ntiles * (blockIdx.x + 1) / gridDim.x;
  const int64_t end = P.pos + P.len;
  const int64_t lo = P.pos + t0 * kStageTile;
  const int64_t hi = P.pos + t1 * kStageTile < end ? P.pos + t1 * kStageTile : end;
  if (lo >= hi) return;
  if (UNPACK) stage_unpack<G, kStageBufs>(P, P.c - P.pos, wt, lo, hi, sbuf, mbar, threadIdx.x, blockDim.x);
  else stage_pack<G, kStageBufs>(P, P.c - P.pos, wt, lo, hi, sbuf, threadIdx.x, blockDim.x);
}

// f1: fused type -> type copies (no packed buffer)
__global__ void __launch_bounds__(256, 3) k_dual_seg(const KP S, const KP R, int64_t n, int64_t per_warp) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t p = gw * per_warp;
  dual_walk(S, R, p, min(p + per_warp, n), lane);
}

template <int G>
__global__ void __launch_bounds__(256) k_dual_stage(const KP S, const KP R, int64_t n, int64_t ntiles) {
  extern __shared__ __align__(128) uint8_t smem_dual[];
  uint8_t* sbuf = smem_dual;
  int32_t* wts = reinterpret_cast<int32_t*>(smem_dual + kStageBufs * kStageTile);
  int32_t* wtr = wts + S.nwords;
  for (int i = threadIdx.x; i < S.nwords; i += blockDim.x) wts[i] = S.wtab[i];
  for (int i = threadIdx.x; i < R.nwords; i += blockDim.x) wtr[i] = R.wtab[i];
  __syncthreads();
  const int64_t t0 = ntiles * blockIdx.x / gridDim.x, t1 = ntiles * (blockIdx.x + 1) / gridDim.x;
  const int64_t lo = t0 * kStageTile, hi = t1 * kStageTile < n ? t1 * kStageTile : n;
  if (lo < hi) stage_copy<G, kStageBufs>(S, wts, R, wtr, lo, hi, sbuf);
}

template <int G>
__global__ void __launch_bounds__(256) k_dual_word(const KP S, const KP R, int64_t n) {
  extern __shared__ int32_t wts[];
  int32_t* wtr = wts + S.nwords;
  for (int i = threadIdx.x; i < S.nwords; i += blockDim.x) wts[i] = S.wtab[i];
  for (int i = threadIdx.x; i < R.nwords; i += blockDim.x) wtr[i] = R.wtab[i];
  __syncthreads();
  dual_words<G, 4>(S, wts, R, wtr, 0, n, (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                   (int64_t)gridDim.x * blockDim.x);
}

// record-span pack/unpack (short blocks in small dense records): warp w takes
// batches w, w + nwarps, ... of RB records
template <bool UNPACK, int G>
__global__ void __launch_bounds__(256, 3) k_rec(const KP P, const RecGeo R) {
  extern __shared__ __align__(16) uint8_t smem_rec[];
  const int nwc = blockDim.x >> 5, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int bufB = R.RB * R.spanB;
  uint8_t* buf = smem_rec + w * bufB;
  int64_t* sd = reinterpret_cast<int64_t*>(smem_rec + nwc * bufB) + w * R.RB;
  uint16_t* omap = reinterpret_cast<uint16_t*>(smem_rec + nwc * bufB + nwc * R.RB * 8);
  rec_maps<UNPACK, G>(R, omap);
  __syncthreads();
  rec_range<UNPACK, G, LD_CS>(P, R, P.c - P.pos, P.pos, P.pos + P.len, buf, sd, omap,
                              (int64_t)blockIdx.x * nwc + w, (int64_t)gridDim.x * nwc, lane);
}

template <bool UNPACK, int G, int VW>
__global__ void __launch_bounds__(256) k_word(const KP P) {
  extern __shared__ int32_t wt[];
  // single-block template: word offsets are arithmetic (no dependent table load
  // before the first gather -- it matters for latency-bound faces, C4 x)
  const bool sb = P.nblocks == 1;
  if (!sb) {
    for (int i = threadIdx.x; i < P.nwords; i += blockDim.x) wt[i] = P.wtab[i];
    __syncthreads();
  }
  word_range<UNPACK, G, VW, LD_CS, (G >= 4 ? 4 : 2)>(P, P.c - P.pos, P.pos, P.pos + P.len, sb ? nullptr : wt,
                                                     (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                                                     (int64_t)gridDim.x * blockDim.x);
}
// --------------------------------------------------------------- host side
// Per-device launch state: kernel attributes (max dynamic smem) are per device, so
// a process driving several devices (dt_comm_connect supports it) sets them on each.
struct DevLaunch {
  int sms = 0;
  bool rec_attr = false, stage_attr = false, span_attr = false, dual_attr = false;
  int span_occ = 0, word_occ = 0;
  int seg_occ[2][2] = {{0, 0}, {0, 0}};
};
static DevLaunch g_devl[64];
static DevLaunch& devl() {
  int dev = 0;
  cudaGetDevice(&dev);
  return g_devl[dev & 63];
}
static int num_sms() {
  DevLaunch& d = devl();
  if (!d.sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev);
    if (d.sms <= 0) d.sms = 148;
  }
  return d.sms;
}

static dt_status cuda_fail(cudaError_t e, const char* what) {
  set_error("%s: %s", what, cudaGetErrorString(e));
  return DT_ERR_CUDA;
}
#define CU(call)                                        \
  do {                                                  \
    cudaError_t _e = (call);                            \
    if (_e != cudaSuccess) return cuda_fail(_e, #call); \
  } while (0)

void free_desc(DeviceDesc& dd) {
  int cur = -1;
  cudaGetDevice(&cur);
  if (dd.device >= 0 && dd.device != cur) cudaSetDevice(dd.device);
  cudaFree(dd.bd);
  cudaFree(dd.bl);
  cudaFree(dd.boff);
  for (auto* p : dd.tables) cudaFree(p);
  for (auto*& w : dd.wtab) { cudaFree(w); w = nullptr; }
  cudaFree(dd.sdesc);
  cudaFree(dd.wbase);
  dd.sdesc = nullptr;
  dd.wbase = nullptr;
  dd.sdesc_state = -1;
  dd.bd = dd.bl = dd.boff = nullptr;
  dd.tables.clear();
  for (auto& sl : dd.plans) {
    cudaFree(sl.d);
    if (sl.ready) cudaEventDestroy((cudaEvent_t)sl.ready);
  }
  dd.plans.clear();
  if (cur >= 0 && dd.device >= 0 && dd.device != cur) cudaSetDevice(cur);
}

static int log2_small(int64_t g) { return g == 1 ? 0 : g == 2 ? 1 : g == 4 ? 2 : g == 8 ? 3 : 4; }

dt_status upload_desc(dt_type_s* t, const Form& f, DeviceDesc& dd) {
  (void)t;
  cudaStream_t s;
  CU(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  const int64_t nb = (int64_t)f.bl.size();
  const size_t bytes = sizeof(int64_t) * (size_t)std::max<int64_t>(nb, 1);
  CU(cudaMalloc(&dd.bd, bytes));
  CU(cudaMalloc(&dd.bl, bytes));
  CU(cudaMalloc(&dd.boff, bytes));
  if (nb > 0) {
    CU(cudaMemcpyAsync(dd.bd, f.bd.data(), sizeof(int64_t) * nb, cudaMemcpyHostToDevice, s));
    CU(cudaMemcpyAsync(dd.bl, f.bl.data(), sizeof(int64_t) * nb, cudaMemcpyHostToDevice, s));
    const int64_t ntile = (nb + kScanTile - 1) / kScanTile;
    int64_t* sums = nullptr;
    CU(cudaMallocAsync(&sums, sizeof(int64_t) * ntile, s));
    k_scan_local<<<(unsigned)ntile, kScanNT, 0, s>>>(dd.bl, dd.boff, sums, nb);
    k_scan_sums<<<1, kScanNT, 0, s>>>(sums, ntile);
    k_scan_add<<<(unsigned)ntile, kScanNT, 0, s>>>(dd.boff, sums, nb);
    CU(cudaGetLastError());
    CU(cudaFreeAsync(sums, s));
  }
  dd.tables.assign(f.lv.size(), nullptr);
  for (size_t i = 0; i < f.lv.size(); i++) {
    if (!f.lv[i].is_list()) continue;
    const auto& tab = *f.lv[i].table;
    CU(cudaMalloc(&dd.tables[i], sizeof(int64_t) * tab.size()));
    CU(cudaMemcpyAsync(dd.tables[i], tab.data(), sizeof(int64_t) * tab.size(), cudaMemcpyHostToDevice, s));
  }
  CU(cudaStreamSynchronize(s));
  // sanity: the device prefix must end at tsize - last len
  if (nb > 0) {
    int64_t last = 0;
    CU(cudaMemcpy(&last, dd.boff + nb - 1, sizeof(int64_t), cudaMemcpyDeviceToHost));
    if (last != f.tsize() - f.bl.back()) {
      set_error("device scan mismatch (%lld vs %lld)", (long long)last, (long long)(f.tsize() - f.bl.back()));
      cudaStreamDestroy(s);
      return DT_ERR_CUDA;
    }
  }
  CU(cudaStreamDestroy(s));
  return DT_OK;
}

// word table of the template at granularity g: word k -> byte offset of its
// source inside the element (int32).  Built lazily per granularity.
static dt_status ensure_wtab(const Form& f, DeviceDesc& dd, int64_t g, const int32_t** out) {
  int li = log2_small(g);
  if (!dd.wtab[li]) {
    if (f.host_missing()) {
      dt_status ms = materialize_host(f, dd);
      if (ms != DT_OK) return ms;
    }
    const int64_t nw = f.tsize() / g;
    std::vector<int32_t> h((size_t)nw);
    int64_t k = 0;
    for (size_t b = 0; b < f.bl.size(); b++)
      for (int64_t o = 0; o < f.bl[b]; o += g) h[(size_t)k++] = (int32_t)(f.bd[b] + o);
    CU(cudaMalloc(&dd.wtab[li], sizeof(int32_t) * std::max<int64_t>(nw, 1)));
    CU(cudaMemcpy(dd.wtab[li], h.data(), sizeof(int32_t) * nw, cudaMemcpyHostToDevice));
  }
  *out = dd.wtab[li];
  return DT_OK;
}

dt_status ensure_wtab_pub(const Form& f, DeviceDesc& dd, int64_t g, const int32_t** out) {
  return ensure_wtab(f, dd, g, out);
}

__global__ void k_build_sdesc(const int64_t* __restrict__ bd, const int64_t* __restrict__ bl, int64_t n,
                              uint64_t* __restrict__ sdesc, int64_t* __restrict__ wbase) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t base = bd[i & ~int64_t(31)];
    if ((i & 31) == 0) wbase[i >> 5] = base;
    sdesc[i] = ((uint64_t)bl[i] << 32) | (uint32_t)(int32_t)(bd[i] - base);
  }
}

dt_status ensure_sdesc(const Form& f, DeviceDesc& dd, const uint64_t** sdesc, const int64_t** wbase) {
  if (dd.sdesc_state < 0) {
    // representable? (host check once per descriptor, O(n))
    const char* no = getenv("DT_NO_SDESC");  // (A/B switch)
    bool ok = !(no && *no && *no != '0');
    const size_t n = (size_t)f.nblocks();
    if (ok && f.sdesc_ok_cache >= 0) {
      ok = f.sdesc_ok_cache == 1;  // (known from the flattening pass)
    } else {
      for (size_t i = 0; i < n && ok; i++) {
        const int64_t r = f.bd[i] - f.bd[i & ~size_t(31)];
        ok = r >= INT32_MIN && r <= INT32_MAX && f.bl[i] < (int64_t(1) << 32) && f.bl[i] >= 0;
      }
    }
    dd.sdesc_state = 0;
    if (ok && n > 1) {
      CU(cudaMalloc(&dd.sdesc, sizeof(uint64_t) * n));
      CU(cudaMalloc(&dd.wbase, sizeof(int64_t) * ((n + 31) / 32)));
      const unsigned grid = (unsigned)std::min<int64_t>((int64_t)(n + 255) / 256, 4096);
      cudaStream_t s;  // a private non-blocking stream: never waits for the caller's work
      CU(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
      k_build_sdesc<<<grid, 256, 0, s>>>(dd.bd, dd.bl, (int64_t)n, dd.sdesc, dd.wbase);
      CU(cudaGetLastError());
      CU(cudaStreamSynchronize(s));  // once per committed type and device
      CU(cudaStreamDestroy(s));
      dd.sdesc_state = 1;
    }
  }
  *sdesc = dd.sdesc_state == 1 ? dd.sdesc : nullptr;
  *wbase = dd.sdesc_state == 1 ? dd.wbase : nullptr;
  return DT_OK;
}

static int64_t lowp2(uint64_t x) {
  if (x == 0) return 16;
  int64_t g = (int64_t)(x & (~x + 1));
  return g > 16 ? 16 : g;
}

// Levels for one launch: the committed form's levels with the instance level
// (count, extent) prepended as the outermost level, merged when regular.
void build_levels(const Form& f, const DeviceDesc* dd, dt_type_s* t, int64_t count, KLevels& L) {
  L.n = 0;
  int off = 0;
  if (count > 1) {
    L.cnt[0] = count;
    L.stride[0] = t->extent();
    L.table[0] = nullptr;
    L.n = 1;
    off = 1;
  }
  for (size_t i = 0; i < f.lv.size(); i++) {
    L.cnt[off + i] = f.lv[i].cnt;
    L.stride[off + i] = f.lv[i].stride;
    L.table[off + i] = f.lv[i].is_list() ? (dd ? dd->tables[i] : reinterpret_cast<const int64_t*>(1)) : nullptr;
    L.n++;
  }
  // merge the instance level into the next regular level when contiguous in index space
  if (count > 1 && L.n >= 2 && !L.table[1] && L.stride[0] == L.cnt[1] * L.stride[1]) {
    L.cnt[1] *= L.cnt[0];
    for (int i = 0; i + 1 < L.n; i++) {
      L.cnt[i] = L.cnt[i + 1];
      L.stride[i] = L.stride[i + 1];
      L.table[i] = L.table[i + 1];
    }
    L.n--;
  }
}

static bool template_fits_int32(const Form& f) {
  if (f.fits32_cache >= 0) return f.fits32_cache == 1;
  if (f.host_missing()) return false;  // (device forms carry the fact)
  f.fits32_cache = 0;
  for (size_t b = 0; b < f.bd.size(); b++)
    if (f.bd[b] < INT32_MIN || f.bd[b] + f.bl[b] > INT32_MAX) return false;
  f.fits32_cache = 1;
  return true;
}

// Effective template of one launch: a single-block template whose innermost
// regular level continues the run (e.g. count instances of a contiguous type)
// becomes one longer run, when that makes it a long-run copy.
Eff effective(const Form& f, const DeviceDesc* dd, dt_type_s* t, int64_t count) {
  Eff E;
  build_levels(f, dd, t, count, E.L);
  E.tsize = f.tsize();
  E.nblocks = f.nblocks();
  E.bd0 = f.first_bd();
  E.bl0 = f.first_bl();
  E.merged = false;
  KLevels& L = E.L;
  while (E.nblocks == 1 && L.n >= 1 && !L.table[L.n - 1] && L.stride[L.n - 1] == E.bl0 &&
         E.bl0 * L.cnt[L.n - 1] >= 256) {
    E.bl0 *= L.cnt[L.n - 1];
    E.tsize = E.bl0;
    L.n--;
    E.merged = true;
  }
  return E;
}

// per-segment fixed cost in byte-equivalents (one round trip at a warp's share of HBM bandwidth)
static int64_t seg_alpha() {
  static const int64_t a = getenv("DT_SEG_ALPHA") ? atoll(getenv("DT_SEG_ALPHA")) : 2048;
  return a;
}

// cost of stream byte p (see PlanEnt): p + alpha * (block starts before it)
static int64_t host_cost(const KP& P, const Form& f, int64_t alpha, int64_t p) {
  const int64_t ce = P.tsize + alpha * P.nblocks;
  const int64_t e = p / P.tsize;
  const int64_t rem = p - e * P.tsize;
  if (rem == 0) return e * ce;  // element boundary (pos 0, a whole stream): no block search
  int64_t b = 0, bo = 0;
  if (P.nblocks > 1) {
    const auto& h = f.hoff();
    b = (int64_t)(std::upper_bound(h.begin(), h.end(), rem) - h.begin()) - 1;
    bo = h[(size_t)b];
  }
  return e * ce + bo + alpha * b + (rem - bo);
}

// cached (or freshly computed) cost-balanced plan for this launch shape
static dt_status get_plan(dt_type_s* t, const KP& P, const Form& f, DeviceDesc& dd, int64_t count, int64_t nw,
                          cudaStream_t s, const PlanEnt** out, int64_t alpha = -1, int64_t gran = 1) {
  if (alpha < 0) alpha = seg_alpha();
  std::lock_guard<std::mutex> g(t->mu);
  for (auto& sl : dd.plans) {
    if (sl.d && sl.count == count && sl.pos == P.pos && sl.len == P.len && sl.nw == nw && sl.alpha == alpha &&
        sl.tsize == P.tsize && sl.gran == gran) {
      // the plan was filled by a kernel on sl.made_on: another stream must wait for it
      if ((void*)s != sl.made_on) CU(cudaStreamWaitEvent(s, (cudaEvent_t)sl.ready, 0));
      *out = (const PlanEnt*)sl.d;
      return DT_OK;
    }
  }
  size_t idx;
  if (dd.plans.size() < 64) {  // (a host-link pipeline uses one plan per chunk)
    dd.plans.emplace_back();
    idx = dd.plans.size() - 1;
  } else {
    idx = dd.plan_next++ % dd.plans.size();
  }
  DeviceDesc::PlanSlot& sl = dd.plans[idx];
  if (sl.d) {  // eviction: cudaFree waits for in-flight users of the old plan
    cudaFree(sl.d);
    sl.d = nullptr;
  }
  sl.count = -1;
  CU(cudaMalloc(&sl.d, sizeof(PlanEnt) * (size_t)(nw + 1)));
  const int64_t ce = P.tsize + alpha * P.nblocks;
  if (f.host_missing() && P.nblocks > 1 && (P.pos % P.tsize || (P.pos + P.len) % P.tsize)) {
    dt_status ms = materialize_host(f, dd);  // (host_cost needs the block prefix)
    if (ms != DT_OK) return ms;
  }
  const int64_t C0 = host_cost(P, f, alpha, P.pos), C1 = host_cost(P, f, alpha, P.pos + P.len);
  k_plan<<<(unsigned)((nw + 1 + 255) / 256), 256, 0, s>>>(P, alpha, make_fd((uint64_t)ce), ce, C0, C1, nw,
                                                          gran, (PlanEnt*)sl.d);
  CU(cudaGetLastError());
  if (!sl.ready) CU(cudaEventCreateWithFlags((cudaEvent_t*)&sl.ready, cudaEventDisableTiming));
  CU(cudaEventRecord((cudaEvent_t)sl.ready, s));
  sl.made_on = (void*)s;
  sl.count = count;
  sl.pos = P.pos;
  sl.len = P.len;
  sl.nw = nw;
  sl.alpha = alpha;
  sl.gran = gran;
  sl.tsize = P.tsize;
  *out = (const PlanEnt*)sl.d;
  return DT_OK;
}

// Record-span geometry of a launch (k_rec), or false when it does not apply:
// G >= 4, 16-byte-aligned element bases and packed side, the template inside a
// 16-byte-aligned span of <= 128 B that is at least half payload.
bool rec_geometry(const Form& f, const KLevels& L, uint64_t nc_addr, uint64_t c_addr, int64_t pos, int64_t len,
                  int64_t g, RecGeo* R) {
  if (g < 4 || f.empty() || len <= 0) return false;
  if ((nc_addr & 15) || ((c_addr - (uint64_t)pos) & 15)) return false;
  int64_t lg = level_granularity(f);
  for (int i = 0; i < L.n; i++)
    if (!L.table[i]) lg = std::min(lg, lowp2((uint64_t)L.stride[i]));
  if (lg < 16) return false;
  if (f.nblocks() > 64) return false;  // (a <= 128-byte span holds few blocks; keeps planning O(1))
  int64_t lo, hi;
  f.span(&lo, &hi);
  const int64_t a0 = lo >= 0 ? lo & ~int64_t(15) : -((-lo + 15) & ~int64_t(15));
  const int64_t spanB = ((hi - a0) + 15) & ~int64_t(15);
  const int64_t ts = f.tsize();
  if (spanB > 128 || 2 * ts < spanB || ts % g) return false;
  R->a0 = a0;
  R->spanB = (int32_t)spanB;
  R->nch = (int32_t)(spanB / 16);
  R->RB = 32 * (8 / R->nch);
  R->LPL = R->RB * R->nch / 32;
  R->nwr = (int32_t)(ts / g);
  R->invnch = (65536 + R->nch - 1) / R->nch;
  R->e_lo = pos / ts;
  R->e_hi = (pos + len + ts - 1) / ts;
  R->b0 = R->e_lo & ~int64_t(31);
  R->nbatch = (R->e_hi - R->b0 + R->RB - 1) / R->RB;
  if (R->nwr > 32) return false;
  int k = 0;
  for (size_t b = 0; b < f.bd.size(); b++)
    for (int64_t o = 0; o < f.bl[b]; o += g) R->woff[k++] = (uint8_t)((f.bd[b] + o - a0) / g);
  return true;
}

// Block-span kernel precondition (cached per form, O(1) per call): the 32-block
// windows of the stream must be local -- at most a few span buffers wide -- else
// they all take the kernel's wide-span fallback and the block-window kernel is
// faster (tools/kind_probe.py, 64 MiB pack: C5b fully shuffled 110 vs 180 us and an
// unsorted record list 49 vs 82 us favour block windows; C5b 104 vs 58, 16-byte
// blocks with spans around 4 KiB 82 vs 40, C5b shuffled within 48 blocks 102 vs 115
// favour / tie with block spans).  Rule: half of the sampled windows within 16 KiB.
// Sampled: 64 windows of the template, or, for templates of < 32 blocks, 64 windows
// of the innermost level (its stride, or consecutive entries of its table).
static bool span_local(const Form& f) {
  if (f.span_local_cache >= 0) return f.span_local_cache != 0;
  if (f.host_missing()) return false;  // (device forms carry the fact)
  const int64_t nb = (int64_t)f.bl.size();
  constexpr int64_t kBuf = 4 * 4096;
  int good = 0, tot = 0;
  if (nb >= 32) {
    for (int s = 0; s < 64; s++) {
      const int64_t i0 = (nb - 32) * s / 63;
      int64_t lo = INT64_MAX, hi = INT64_MIN;
      for (int64_t i = i0; i < i0 + 32; i++) {
        lo = std::min(lo, f.bd[(size_t)i]);
        hi = std::max(hi, f.bd[(size_t)i] + f.bl[(size_t)i]);
      }
      tot++;
      good += hi - lo <= kBuf;
    }
  } else if (!f.lv.empty()) {
    int64_t tlo, thi;
    f.span(&tlo, &thi);
    const int64_t tspan = thi - tlo, epw = (32 + nb - 1) / nb;  // elements per window
    const Level& in = f.lv.back();
    if (!in.is_list()) {
      tot = 1;
      good = (int)(std::llabs(in.stride) * (epw - 1) + tspan <= kBuf);
    } else {
      const std::vector<int64_t>& tb = *in.table;
      const int64_t n = (int64_t)tb.size();
      for (int s = 0; s < 64; s++) {
        const int64_t i0 = std::max<int64_t>(0, n - epw) * s / 63;
        int64_t lo = INT64_MAX, hi = INT64_MIN;
        for (int64_t i = i0; i < std::min(n, i0 + epw); i++) {
          lo = std::min(lo, tb[(size_t)i]);
          hi = std::max(hi, tb[(size_t)i]);
        }
        tot++;
        good += hi - lo + tspan <= kBuf;
      }
    }
  } else {
    tot = good = 1;  // one small template: instances at the extent (dense for these lists)
  }
  f.span_local_cache = good * 2 >= tot ? 1 : 0;
  return f.span_local_cache != 0;
}

int plan_kernel(const Form& f, const KLevels& L, uint64_t nc_addr, uint64_t c_addr, int64_t pos, int64_t len,
                int64_t* gran) {
  if (len <= 0 || f.empty()) return 0;
  const int64_t nb = f.nblocks();
  const int64_t ts = f.tsize();
  int64_t g = form_granularity(f);
  for (int i = 0; i < L.n; i++)
    if (!L.table[i]) g = std::min(g, lowp2((uint64_t)L.stride[i]));  // list tables counted in form
  g = std::min(g, lowp2(nc_addr));
  g = std::min(g, lowp2(c_addr));
  g = std::min(g, lowp2((uint64_t)pos));
  g = std::min(g, lowp2((uint64_t)len));
  *gran = g;
  const double mean = (double)ts / (double)nb;
  const bool word_ok = ts / g <= kMaxWordTable && ts % g == 0 && template_fits_int32(f);
  const char* fk = getenv("DT_FORCE_KERNEL");  // tuning / test aid: force a kernel family when applicable
  const int force = fk ? atoi(fk) : 0;
  const bool blk_ok = (c_addr & 15) == 0 && ts % g == 0;
  const bool stage_ok = word_ok && g >= 4 && (c_addr & 15) == 0;
  RecGeo rg;
  const bool rec_ok = rec_geometry(f, L, nc_addr, c_addr, pos, len, g, &rg);
  if (force == 6 && rec_ok) return 6;
  if (force == 2 && word_ok) return 2;
  if (force == 3 && blk_ok) return 3;
  if (force == 7 && g >= 4) return 7;
  if (force == 4 && stage_ok) return 4;
  if (force == 1) return 1;
  // short blocks / co-aligned runs up to 1 KiB: with >= 8-byte words the smem/TMA
  // staged kernel wins (C3 pack 0.78 of copy vs 0.66 word table vs 0.44 warp
  // segments; measured), with 4-byte words the register word kernel does
  // short blocks in small dense records (C5 particles): whole-record 16-byte loads
  if (mean < 256.0 && rec_ok && !force) return 6;
  if ((mean < 256.0 || (g == 16 && mean < 1024.0)) && word_ok) return stage_ok && g >= stage_min_g() ? 4 : 2;
  // many short blocks (no word table): block spans with >= 4-byte words, else block windows
  if (mean < 128.0 && g >= 4 && !force && span_local(f)) return 7;
  if (mean < 128.0 && blk_ok) return 3;
  return 1;
}

static int seg_occupancy(bool unpack, bool single) {
  int& o = devl().seg_occ[unpack][single];
  if (!o) {
    const void* f = unpack ? (single ? (const void*)k_seg<true, true> : (const void*)k_seg<true, false>)
                           : (single ? (const void*)k_seg<false, true> : (const void*)k_seg<false, false>);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, f, 256, 0) != cudaSuccess || o < 1) o = 4;
  }
  return o;
}

template <bool UNPACK>
static void launch_word(const KP& P, int64_t g, bool vec16, unsigned grid, size_t smem, cudaStream_t s) {
#define LW(G, VW) k_word<UNPACK, G, VW><<<grid, 256, smem, s>>>(P)
  if (vec16) {
    switch (g) {
      case 1: LW(1, 16); break;
      case 2: LW(2, 16); break;
      case 4: LW(4, 16); break;
      case 8: LW(8, 16); break;
      default: LW(16, 16); break;
    }
  } else {
    switch (g) {
      case 1: LW(1, 1); break;
      case 2: LW(2, 2); break;
      case 4: LW(4, 4); break;
      case 8: LW(8, 8); break;
      default: LW(16, 16); break;
    }
  }
#undef LW
}

dt_status launch_pack_unpack(bool unpack, dt_type_s* t, const Form& f, DeviceDesc& dd, int64_t count, const void* nc,
                             void* c, int64_t pos, int64_t len, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  Eff E = effective(f, &dd, t, count);
  const KLevels& L = E.L;
  KP P;
  std::memset(&P, 0, sizeof(P));
  P.nc = (const uint8_t*)nc;
  P.c = (uint8_t*)c;
  P.pos = pos;
  P.len = len;
  P.tsize = E.tsize;
  P.nblocks = E.nblocks;
  P.bd = dd.bd;
  P.bl = dd.bl;
  P.boff = dd.boff;
  P.bd0 = E.bd0;
  P.bl0 = E.bl0;
  P.nlev = L.n;
  for (int i = 0; i < L.n; i++) {
    P.cnt[i] = L.cnt[i];
    P.stride[i] = L.stride[i];
    P.table[i] = L.table[i];
    P.fcnt[i] = make_fd((uint64_t)L.cnt[i]);
  }
  P.ftsize = make_fd((uint64_t)P.tsize);
  int64_t g = 1;
  int kind = E.merged ? 1 : plan_kernel(f, L, (uint64_t)(uintptr_t)nc, (uint64_t)(uintptr_t)c, pos, len, &g);
  if (kind == 0) return DT_OK;
  // grids are sized in SMs' worth of resident CTAs; DT_MAX_SMS caps it (f3: how few
  // SMs a pack/unpack needs, e.g. to leave the rest to a co-running application)
  const char* ms = getenv("DT_MAX_SMS");
  const int sms = ms && atoi(ms) > 0 ? std::min(num_sms(), atoi(ms)) : num_sms();
  if (kind == 6) {
    RecGeo R;
    if (!rec_geometry(f, L, (uint64_t)(uintptr_t)nc, (uint64_t)(uintptr_t)c, pos, len, g, &R)) {
      set_error("record-span geometry changed between plan and launch");
      return DT_ERR_ARG;
    }
    P.nwords = R.nwr;
    const int nwc = 8;
    const size_t tabB = std::max<size_t>((size_t)R.RB * R.nwr * 2, (size_t)(R.spanB / g) * 2);
    const size_t smem = (size_t)nwc * R.RB * R.spanB + (size_t)nwc * R.RB * 8 + ((tabB + 15) & ~size_t(15));
    bool& attr = devl().rec_attr;
    if (!attr) {
      const void* fs[] = {(const void*)k_rec<false, 4>, (const void*)k_rec<false, 8>, (const void*)k_rec<false, 16>,
                          (const void*)k_rec<true, 4>,  (const void*)k_rec<true, 8>,  (const void*)k_rec<true, 16>};
      for (const void* fp : fs) cudaFuncSetAttribute(fp, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
      attr = true;
    }
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_rec<false, 4>, 256, smem) != cudaSuccess || occ < 1)
      occ = 1;
    const int64_t need = (R.nbatch + nwc - 1) / nwc;
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * occ, need));
#define LR(U, G) k_rec<U, G><<<grid, 256, smem, s>>>(P, R)
    if (unpack) {
      switch (g) { case 4: LR(true, 4); break; case 8: LR(true, 8); break; default: LR(true, 16); break; }
    } else {
      switch (g) { case 4: LR(false, 4); break; case 8: LR(false, 8); break; default: LR(false, 16); break; }
    }
#undef LR
  } else if (kind == 1 && P.nblocks == 1 && P.nlev == 0 && !getenv("DT_NO_RUN_COPY") &&
             !(((uintptr_t)(P.nc + P.bd0 + pos) | (uintptr_t)c | (uint64_t)len) & 15)) {
    const uint4* src = reinterpret_cast<const uint4*>(unpack ? (const uint8_t*)c : P.nc + P.bd0 + pos);
    uint4* dst = reinterpret_cast<uint4*>(unpack ? const_cast<uint8_t*>(P.nc) + P.bd0 + pos : (uint8_t*)c);
    const int64_t nv = len / 16;
    const int64_t per_cta = 128 * 4;
    const unsigned grid = (unsigned)std::min<int64_t>((nv + per_cta - 1) / per_cta, (int64_t)sms * 64);
    k_run_copy<<<grid, 128, 0, s>>>(src, dst, nv);
  } else if (kind == 1 && P.nblocks == 1) {
    // one wave of resident CTAs, equal 16-byte-multiple slices of >= 1 KiB per warp
    const int occ = seg_occupancy(unpack, true);
    const int64_t max_warps = (int64_t)sms * occ * 8;
    int64_t per = std::max<int64_t>(1024, (len + max_warps - 1) / max_warps);
    if (per > (int64_t(128) << 10)) per = 16384;  // long streams: several waves of 16 KiB slices (as k_seg)
    per = (per + 15) & ~int64_t(15);
    const int64_t nw = (len + per - 1) / per;
    const unsigned grid = (unsigned)((nw + 7) / 8);
    if (unpack) k_seg_eq<true><<<grid, 256, 0, s>>>(P, per);
    else k_seg_eq<false><<<grid, 256, 0, s>>>(P, per);
  } else if (kind == 1) {
    // exactly one wave of resident CTAs (no tail wave), at least ~4 KiB per warp
    const bool single = P.nblocks == 1;
    const int occ = seg_occupancy(unpack, single);
    const int64_t max_warps = (int64_t)sms * occ * 8;
    int64_t nw = std::min<int64_t>(max_warps, std::max<int64_t>(1, (len + 4095) / 4096));
    // Long streams: when one wave would give each warp more than 128 KiB, cut 16 KiB slices
    // instead and let several waves of short CTAs take them -- neighbouring warps then work
    // on neighbouring stream bytes (T16K 1 GiB: 0.935 of the same-run copy vs 0.877 with
    // one wave; T8K, 75 KiB per warp, unchanged).  DT_SEG_SLICE=<bytes> forces a slice size.
    const char* se = getenv("DT_SEG_SLICE");
    const int64_t slice = se && atoll(se) > 0 ? atoll(se) : (len > max_warps * (int64_t(128) << 10) ? 16384 : 0);
    if (slice > 0) nw = std::max<int64_t>(1, (len + slice - 1) / slice);
    const PlanEnt* plan = nullptr;
    dt_status pst = get_plan(t, P, f, dd, count, nw, s, &plan);
    if (pst != DT_OK) return pst;
    unsigned grid = (unsigned)((nw + 7) / 8);
    if (unpack) {
      if (single) k_seg<true, true><<<grid, 256, 0, s>>>(P, plan, nw);
      else k_seg<true, false><<<grid, 256, 0, s>>>(P, plan, nw);
    } else {
      if (single) k_seg<false, true><<<grid, 256, 0, s>>>(P, plan, nw);
      else k_seg<false, false><<<grid, 256, 0, s>>>(P, plan, nw);
    }
  } else if (kind == 4) {
    const int32_t* wt = nullptr;
    dt_status st = ensure_wtab(f, dd, g, &wt);
    if (st != DT_OK) return st;
    P.wtab = wt;
    P.nwords = (int32_t)(f.tsize() / g);
    const size_t smem = (size_t)kStageBufs * kStageTile + sizeof(int32_t) * (size_t)P.nwords;
    const int64_t ntiles = (len + kStageTile - 1) / kStageTile;
    bool& attr_set = devl().stage_attr;
    if (!attr_set) {
      const void* fs[] = {(const void*)k_stage<false, 4>, (const void*)k_stage<false, 8>,
                          (const void*)k_stage<false, 16>, (const void*)k_stage<true, 4>,
                          (const void*)k_stage<true, 8>, (const void*)k_stage<true, 16>};
      for (const void* fp : fs) cudaFuncSetAttribute(fp, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
      attr_set = true;
    }
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_stage<false, 4>, 256, smem) != cudaSuccess || occ < 1)
      occ = 1;
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * occ, ntiles));
#define LS(U, G) k_stage<U, G><<<grid, 256, smem, s>>>(P, ntiles)
    if (unpack) {
      switch (g) { case 4: LS(true, 4); break; case 8: LS(true, 8); break; default: LS(true, 16); break; }
    } else {
      switch (g) { case 4: LS(false, 4); break; case 8: LS(false, 8); break; default: LS(false, 16); break; }
    }
#undef LS
  } else if (kind == 7) {
    P.fnb = make_fd((uint64_t)P.nblocks);
    {
      dt_status sst = ensure_sdesc(f, dd, &P.sdesc, &P.wbase);
      if (sst != DT_OK) return sst;
    }
    const size_t smem = 8 * (size_t)kSpanWarpSmem;
    bool& attr = devl().span_attr;
    if (!attr) {
      const void* fs[] = {(const void*)k_span<false, 4>, (const void*)k_span<false, 8>, (const void*)k_span<false, 16>,
                          (const void*)k_span<true, 4>,  (const void*)k_span<true, 8>,  (const void*)k_span<true, 16>};
      for (const void* fp : fs) cudaFuncSetAttribute(fp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      attr = true;
    }
    int& occ = devl().span_occ;
    if (!occ && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_span<false, 4>, 256, smem) != cudaSuccess ||
                 occ < 1))
      occ = 1;
    // equal byte slices (alpha 0) cut at word boundaries, resolved once per launch
    // shape by k_plan and cached on the type (no per-warp block search)
    const int64_t max_warps = (int64_t)sms * occ * 8;
    const int64_t nw = std::min<int64_t>(max_warps, std::max<int64_t>(1, (len + 4095) / 4096));
    const PlanEnt* plan = nullptr;
    dt_status pst = get_plan(t, P, f, dd, count, nw, s, &plan, 0, g);
    if (pst != DT_OK) return pst;
    const unsigned grid = (unsigned)((nw + 7) / 8);
#define LP(U, G) k_span<U, G><<<grid, 256, smem, s>>>(P, plan, nw)
    if (unpack) {
      switch (g) { case 4: LP(true, 4); break; case 8: LP(true, 8); break; default: LP(true, 16); break; }
    } else {
      switch (g) { case 4: LP(false, 4); break; case 8: LP(false, 8); break; default: LP(false, 16); break; }
    }
#undef LP
  } else if (kind == 3) {
    P.fnb = make_fd((uint64_t)P.nblocks);
    const int64_t max_warps = (int64_t)sms * 4 * 8;
    int64_t nw = std::min<int64_t>(max_warps, std::max<int64_t>(1, (len + 4095) / 4096));
    int64_t per = (len + nw - 1) / nw;
    per = (per + kBlkWin - 1) / kBlkWin * kBlkWin;
    nw = (len + per - 1) / per;
    P.per_warp = per;
    unsigned grid = (unsigned)((nw + 7) / 8);
    size_t smem = 8 * (kBlkWin / g) * sizeof(int64_t);
#define LB(U, G) k_blk<U, G><<<grid, 256, smem, s>>>(P)
    if (unpack) {
      switch (g) { case 1: LB(true, 1); break; case 2: LB(true, 2); break; case 4: LB(true, 4); break;
                   case 8: LB(true, 8); break; default: LB(true, 16); break; }
    } else {
      switch (g) { case 1: LB(false, 1); break; case 2: LB(false, 2); break; case 4: LB(false, 4); break;
                   case 8: LB(false, 8); break; default: LB(false, 16); break; }
    }
#undef LB
  } else {
    const int32_t* wt = nullptr;
    dt_status st = ensure_wtab(f, dd, g, &wt);
    if (st != DT_OK) return st;
    P.wtab = wt;
    P.nwords = (int32_t)(f.tsize() / g);
    const bool vec16 = (((uintptr_t)c) & 15) == 0;
    const int64_t vw = vec16 ? 16 : g;
    const int64_t nvec = (len + vw - 1) / vw;
    size_t smem = sizeof(int32_t) * (size_t)P.nwords;
    // one wave of resident CTAs (grid-stride loop inside)
    int& occ_w = devl().word_occ;
    if (!occ_w && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_w, k_word<false, 4, 16>, 256, 4096) !=
                       cudaSuccess || occ_w < 1))
      occ_w = 4;
    const int64_t maxg = (int64_t)sms * occ_w;
    unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(maxg, (nvec + 255) / 256));
    if (unpack) launch_word<true>(P, g, vec16, grid, smem, s);
    else launch_word<false>(P, g, vec16, grid, smem, s);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
  return DT_OK;
}

dt_status ensure_committed_on_device(dt_type_s* t, DeviceDesc** out) {
  int dev = 0;
  CU(cudaGetDevice(&dev));
  const Form& f = get_form(t);
  std::lock_guard<std::mutex> g(t->mu);
  for (auto& dd : t->devs)
    if (dd.device == dev) { *out = &dd; return DT_OK; }
  if (f.host_missing()) {  // device-flattened on another device: its host arrays first
    dt_status ms = t->devs.empty() ? DT_ERR_ARG : materialize_host(f, t->devs[0]);
    if (ms != DT_OK) return ms;
  }
  t->devs.emplace_back();
  DeviceDesc& dd = t->devs.back();
  dd.device = dev;
  dt_status st = upload_desc(t, f, dd);
  if (st != DT_OK) {
    free_desc(dd);
    t->devs.pop_back();
    return st;
  }
  *out = &dd;
  return DT_OK;
}

static dt_status materialize_t(dt_type_s* t, const Form& f);

// Unpack legality (reading A9): the typemap of `count` instances must not
// overlap.  Cheap structural proof first, exact sorted-interval check if needed.
static int check_nonoverlap(dt_type_s* t, const Form& f, int64_t count) {
  if (f.empty() || count == 0) return 1;
  std::vector<std::pair<int64_t, int64_t>> iv;
  int64_t lo = 0, hi = 0;
  if (f.host_missing() && f.mono_dev == 1) {
    f.span(&lo, &hi);  // device form: the flattening pass proved the blocks sorted and disjoint
  } else {
    if (materialize_t(t, f) != DT_OK) return -1;
    // template: sorted intervals
    iv.reserve(f.bl.size());
    for (size_t i = 0; i < f.bl.size(); i++) iv.push_back({f.bd[i], f.bd[i] + f.bl[i]});
    std::sort(iv.begin(), iv.end());
    for (size_t i = 1; i < iv.size(); i++)
      if (iv[i].first < iv[i - 1].second) return 0;
    lo = iv.front().first;
    for (auto& x : iv) hi = std::max(hi, x.second);
  }
  bool proven = true;
  auto level = [&](int64_t cnt, int64_t stride, const std::vector<int64_t>* tab) {
    if (!proven || cnt <= 1) return;
    const int64_t span = hi - lo;
    if (tab) {
      // index lists are usually sorted (LAMMPS-style): check in place, sort a copy otherwise
      std::vector<int64_t> copy;
      const std::vector<int64_t>* sp = tab;
      if (!std::is_sorted(tab->begin(), tab->end())) {
        copy = *tab;
        std::sort(copy.begin(), copy.end());
        sp = &copy;
      }
      const std::vector<int64_t>& s = *sp;
      for (size_t i = 1; i < s.size(); i++)
        if (s[i] - s[i - 1] < span) { proven = false; return; }
      lo += s.front();
      hi += s.back();
    } else {
      if ((stride < 0 ? -stride : stride) < span) { proven = false; return; }
      int64_t last = (cnt - 1) * stride;
      lo += std::min<int64_t>(0, last);
      hi += std::max<int64_t>(0, last);
    }
  };
  for (int i = (int)f.lv.size() - 1; i >= 0; i--) level(f.lv[i].cnt, f.lv[i].stride, f.lv[i].table.get());
  level(count, t->extent(), nullptr);
  if (proven) return 1;
  if (materialize_t(t, f) != DT_OK) return -1;
  // exact check on the expanded list
  Form g = f;
  if (count > 1) {
    Level l;
    l.cnt = count;
    l.stride = t->extent();
    g.lv.insert(g.lv.begin(), l);
  }
  std::vector<int64_t> d, len;
  if (!expand(g, d, len, int64_t(1) << 26)) return -1;
  iv.clear();
  for (size_t i = 0; i < d.size(); i++) iv.push_back({d[i], d[i] + len[i]});
  std::sort(iv.begin(), iv.end());
  for (size_t i = 1; i < iv.size(); i++)
    if (iv[i].first < iv[i - 1].second) return 0;
  return 1;
}

static dt_status check_dev_ptr(const void* p, const char* what) {
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    set_error("%s: not a device pointer (%s)", what, cudaGetErrorString(e));
    return DT_ERR_ARG;
  }
  if (a.type != cudaMemoryTypeDevice && a.type != cudaMemoryTypeManaged) {
    set_error("%s: host pointer passed to a device entry point (no CPU fallback)", what);
    return DT_ERR_ARG;
  }
  return DT_OK;
}

static bool g_check_ptrs = true;

// pinned host memory the device can address directly (UVA: the same pointer)
static bool host_mapped(const void* p, void** dptr) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  if (a.type != cudaMemoryTypeHost || !a.devicePointer) return false;
  *dptr = a.devicePointer;
  return true;
}

// ------------------------------------------------------- f2: GPU-side flattening
// A huge block list -- an hindexed list of a contiguous element (d0, l0) with per-entry
// counts, the C5b shape -- is flattened ON THE DEVICE at commit (the
// paper prepares its DEV lists on the CPU and pipelines that with the kernels,
// [L18:c1121]-[L18:c1649 §3.2]; here the preparation itself moves to the GPU).  Only the
// raw entry arrays cross the host link; four passes build what the host flattening
// builds -- entry i opens a new block unless it starts where entry i-1 ends (adjacent
// blocks merged, the DEV list of [L16:c5201 §3.2] in typemap order) -- plus the stream
// prefix boff, the compact span descriptors and every fact launch planning asks of the
// form (granularity, span, 32-bit fit, sorted-disjoint, window locality).
//   k_flat_tiles  per 1024-entry tile: sum of lengths, number of block heads, zero count
//   k_scan_sums   exclusive scans of the tile sums (lengths; heads) -> tile offsets
//   k_flat_emit   re-derives each entry's (length, head) and its in-tile prefix; a head
//                 writes bd[o] = disp, boff[o] = stream offset, o = heads before it
//   k_flat_fin    bl[o] = boff[o+1] - boff[o]; descriptors and facts (atomics)
//   k_flat_win    the 64 sampled 32-block windows of span_local()
// Entries of count 0 would make "the previous entry" ambiguous: the pass reports them
// and the commit takes the host flattening instead.  The host arrays of the form are
// downloaded only if a host consumer needs them (materialize_host).
struct FlatFacts {
  unsigned long long orr;  // OR of every merged disp and length
  long long lo, hi;        // min disp, max disp + len
  int not_sdesc, not_mono, zeros, span_good;
  long long bl0;
};

__device__ __forceinline__ void flat_entry(const int64_t* __restrict__ D, const int64_t* __restrict__ B, int64_t i,
                                           int64_t l0, int64_t* l, int64_t* h, int* z) {
  const int64_t b = B[i];
  *l = b * l0;
  *z += b <= 0;
  *h = i == 0 || D[i - 1] + B[i - 1] * l0 != D[i];  // (d0 cancels)
}

__global__ void __launch_bounds__(kScanNT) k_flat_tiles(const int64_t* __restrict__ D, const int64_t* __restrict__ B,
                                                        int64_t n, int64_t l0, int64_t* __restrict__ sl,
                                                        int64_t* __restrict__ sh, FlatFacts* F) {
  const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
  int64_t a = 0, c = 0;
  int z = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; k++) {
    if (base + k >= n) break;
    int64_t l, h;
    flat_entry(D, B, base + k, l0, &l, &h, &z);
    a += l;
    c += h;
  }
  int64_t ta, tc;
  block_exclusive_scan<kScanNT>(a, &ta);
  block_exclusive_scan<kScanNT>(c, &tc);
  if (threadIdx.x == 0) {
    sl[blockIdx.x] = ta;
    sh[blockIdx.x] = tc;
  }
  if (z) atomicAdd(&F->zeros, z);
}

__global__ void __launch_bounds__(kScanNT) k_flat_emit(const int64_t* __restrict__ D, const int64_t* __restrict__ B,
                                                       int64_t n, int64_t d0, int64_t l0,
                                                       const int64_t* __restrict__ sl, const int64_t* __restrict__ sh,
                                                       int64_t* __restrict__ bd, int64_t* __restrict__ boff) {
  const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
  int64_t l[kScanItems], h[kScanItems], a = 0, c = 0;
  int z = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; k++) {
    l[k] = h[k] = 0;
    if (base + k < n) flat_entry(D, B, base + k, l0, &l[k], &h[k], &z);
    a += l[k];
    c += h[k];
  }
  int64_t ta, tc;
  int64_t L = sl[blockIdx.x] + block_exclusive_scan<kScanNT>(a, &ta);
  int64_t H = sh[blockIdx.x] + block_exclusive_scan<kScanNT>(c, &tc);
#pragma unroll
  for (int k = 0; k < kScanItems; k++) {
    if (h[k]) {
      bd[H] = D[base + k] + d0;
      boff[H] = L;
    }
    H += h[k];
    L += l[k];
  }
}

__global__ void __launch_bounds__(256) k_flat_fin(const int64_t* __restrict__ bd, const int64_t* __restrict__ boff,
                                                  int64_t nb, int64_t total, int64_t* __restrict__ bl,
                                                  uint64_t* __restrict__ sdesc, int64_t* __restrict__ wbase,
                                                  FlatFacts* F) {
  unsigned long long orr = 0;
  long long lo = LLONG_MAX, hi = LLONG_MIN;
  int bad_s = 0, bad_m = 0;
  for (int64_t o = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; o < nb; o += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = bd[o];
    const int64_t l = (o + 1 < nb ? boff[o + 1] : total) - boff[o];
    bl[o] = l;
    if (o == 0) F->bl0 = l;
    orr |= (unsigned long long)d | (unsigned long long)l;
    lo = min(lo, (long long)d);
    hi = max(hi, (long long)(d + l));
    if (o + 1 < nb && d + l > bd[o + 1]) bad_m = 1;
    const int64_t gb = bd[o & ~int64_t(31)];
    if ((o & 31) == 0) wbase[o >> 5] = gb;
    const int64_t r = d - gb;
    bad_s |= r < INT32_MIN || r > INT32_MAX || l >= (int64_t(1) << 32);
    sdesc[o] = ((uint64_t)l << 32) | (uint32_t)(int32_t)r;
  }
  // warp reduce, then one atomic per warp
  for (int x = 16; x; x >>= 1) {
    orr |= __shfl_xor_sync(0xffffffffu, orr, x);
    lo = min(lo, (long long)__shfl_xor_sync(0xffffffffu, lo, x));
    hi = max(hi, (long long)__shfl_xor_sync(0xffffffffu, hi, x));
    bad_s |= __shfl_xor_sync(0xffffffffu, bad_s, x);
    bad_m |= __shfl_xor_sync(0xffffffffu, bad_m, x);
  }
  if ((threadIdx.x & 31) == 0) {
    if (orr) atomicOr(&F->orr, orr);
    if (lo != LLONG_MAX) atomicMin(&F->lo, lo);
    if (hi != LLONG_MIN) atomicMax(&F->hi, hi);
    if (bad_s) atomicOr(&F->not_sdesc, 1);
    if (bad_m) atomicOr(&F->not_mono, 1);
  }
}

// span_local()'s sample: window s = blocks [(nb-32)*s/63, +32) within 16 KiB
__global__ void k_flat_win(const int64_t* __restrict__ bd, const int64_t* __restrict__ bl, int64_t nb, FlatFacts* F) {
  const int s = blockIdx.x * 32 + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  const int64_t i = (nb - 32) * s / 63 + lane;
  long long lo = bd[i], hi = bd[i] + bl[i];
  for (int x = 16; x; x >>= 1) {
    lo = min(lo, (long long)__shfl_xor_sync(0xffffffffu, lo, x));
    hi = max(hi, (long long)__shfl_xor_sync(0xffffffffu, hi, x));
  }
  if (lane == 0 && hi - lo <= 4 * 4096) atomicAdd(&F->span_good, 1);
}

// Host -> device copy of several equally long pageable arrays through a process-wide
// pinned double buffer (2 x 16 MiB, allocated once): per chunk, host threads copy into one
// half (memcpy on 8 threads) while the copy engine drains the other; the call returns
// when every chunk is enqueued (the device copies complete in stream order on s).
static dt_status upload_pinned(std::initializer_list<std::pair<const void*, void*>> arrays, size_t bytes,
                               cudaStream_t s) {
  constexpr size_t kHalf = size_t(16) << 20;
  static std::mutex mu;
  static uint8_t* pin = nullptr;
  static cudaEvent_t ev[2] = {nullptr, nullptr};
  std::lock_guard<std::mutex> g(mu);
  if (!pin) {
    CU(cudaHostAlloc((void**)&pin, 2 * kHalf, cudaHostAllocPortable));
    CU(cudaEventCreateWithFlags(&ev[0], cudaEventDisableTiming));
    CU(cudaEventCreateWithFlags(&ev[1], cudaEventDisableTiming));
    CU(cudaEventRecord(ev[0], s));
    CU(cudaEventRecord(ev[1], s));
  }
  int k = 0;
  for (const auto& a : arrays) {
    for (size_t o = 0; o < bytes; o += kHalf, k ^= 1) {
      const size_t m = std::min(kHalf, bytes - o);
      uint8_t* buf = pin + (size_t)k * kHalf;
      CU(cudaEventSynchronize(ev[k]));  // the copy that last read this half is done
      const uint8_t* src = (const uint8_t*)a.first + o;
      constexpr int kT = 8;
      std::thread th[kT];
      const size_t per = ((m + kT - 1) / kT + 63) & ~size_t(63);
      for (int t = 0; t < kT; t++) {
        const size_t lo = std::min(m, (size_t)t * per), hi = std::min(m, lo + per);
        if (lo < hi) th[t] = std::thread([=] { std::memcpy(buf + lo, src + lo, hi - lo); });
      }
      for (auto& x : th)
        if (x.joinable()) x.join();
      CU(cudaMemcpyAsync((uint8_t*)a.second + o, buf, m, cudaMemcpyHostToDevice, s));
      CU(cudaEventRecord(ev[k], s));
    }
  }
  return DT_OK;
}

// DT_OK: flattened and installed; DT_ERR_ARG with *fallback: an entry of count 0 (the
// host flattening handles it); other errors are errors
static dt_status gpu_flatten(dt_type_s* t, int64_t d0, int64_t l0, bool* fallback) {
  *fallback = false;
  const std::vector<int64_t>& B = t->bls;
  const std::vector<int64_t>& Dv = *t->hdps;
  const int64_t n = (int64_t)B.size();
  int dev = 0;
  CU(cudaGetDevice(&dev));
  const int64_t nt = (n + kScanTile - 1) / kScanTile;
  DeviceDesc dd;
  dd.device = dev;
  int64_t *D = nullptr, *Bd = nullptr, *sl = nullptr, *sh = nullptr;
  FlatFacts* F = nullptr;
  FlatFacts h;
  cudaStream_t s = nullptr;
  dt_status st = DT_OK;
  int64_t nb = 0, tot[2] = {0, 0};
  auto fail = [&](cudaError_t e, const char* what) {
    set_error("GPU flattening: %s: %s", what, cudaGetErrorString(e));
    return DT_ERR_CUDA;
  };
#define FU(call)                                                  \
  do {                                                            \
    cudaError_t _e = (call);                                      \
    if (_e != cudaSuccess) { st = fail(_e, #call); goto out; }    \
  } while (0)
  FU(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  FU(cudaMallocAsync(&D, sizeof(int64_t) * n, s));
  FU(cudaMallocAsync(&Bd, sizeof(int64_t) * n, s));
  FU(cudaMallocAsync(&sl, sizeof(int64_t) * (nt + 1), s));
  FU(cudaMallocAsync(&sh, sizeof(int64_t) * (nt + 1), s));
  FU(cudaMallocAsync(&F, sizeof(FlatFacts), s));
  std::memset(&h, 0, sizeof(h));
  h.lo = LLONG_MAX;
  h.hi = LLONG_MIN;
  FU(cudaMemcpyAsync(F, &h, sizeof(h), cudaMemcpyHostToDevice, s));
  {
    // the raw entry arrays through a pinned double buffer: host threads copy a 16 MiB
    // chunk into one half while the copy engine moves the other (a pageable copy of the
    // 480 MB of a 3e7-entry list measured 54-465 ms; the pinned pipeline is bound by the
    // parallel host memcpy)
    st = upload_pinned({{(const void*)Dv.data(), (void*)D}, {(const void*)B.data(), (void*)Bd}},
                       sizeof(int64_t) * (size_t)n, s);
    if (st != DT_OK) goto out;
  }
  k_flat_tiles<<<(unsigned)nt, kScanNT, 0, s>>>(D, Bd, n, l0, sl, sh, F);
  FU(cudaMemsetAsync(sl + nt, 0, sizeof(int64_t), s));
  FU(cudaMemsetAsync(sh + nt, 0, sizeof(int64_t), s));
  k_scan_sums<<<1, kScanNT, 0, s>>>(sl, nt + 1);
  k_scan_sums<<<1, kScanNT, 0, s>>>(sh, nt + 1);
  FU(cudaGetLastError());
  FU(cudaMemcpyAsync(&tot[0], sl + nt, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  FU(cudaMemcpyAsync(&tot[1], sh + nt, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  FU(cudaMemcpyAsync(&h, F, sizeof(h), cudaMemcpyDeviceToHost, s));
  FU(cudaStreamSynchronize(s));
  if (h.zeros) {
    *fallback = true;
    st = DT_ERR_ARG;
    goto out;
  }
  nb = tot[1];
  if (tot[0] != t->size || nb < 1 || nb > n) {
    set_error("GPU flattening: %lld bytes in %lld blocks (type size %lld)", (long long)tot[0], (long long)nb,
              (long long)t->size);
    st = DT_ERR_CUDA;
    goto out;
  }
  FU(cudaMalloc(&dd.bd, sizeof(int64_t) * nb));
  FU(cudaMalloc(&dd.bl, sizeof(int64_t) * nb));
  FU(cudaMalloc(&dd.boff, sizeof(int64_t) * nb));
  FU(cudaMalloc(&dd.sdesc, sizeof(uint64_t) * nb));
  FU(cudaMalloc(&dd.wbase, sizeof(int64_t) * ((nb + 31) / 32)));
  k_flat_emit<<<(unsigned)nt, kScanNT, 0, s>>>(D, Bd, n, d0, l0, sl, sh, dd.bd, dd.boff);
  k_flat_fin<<<(unsigned)std::min<int64_t>((nb + 255) / 256, (int64_t)num_sms() * 8), 256, 0, s>>>(
      dd.bd, dd.boff, nb, tot[0], dd.bl, dd.sdesc, dd.wbase, F);
  if (nb >= 32) k_flat_win<<<2, 32 * 32, 0, s>>>(dd.bd, dd.bl, nb, F);
  FU(cudaGetLastError());
  FU(cudaMemcpyAsync(&h, F, sizeof(h), cudaMemcpyDeviceToHost, s));
  FU(cudaStreamSynchronize(s));
out:
#undef FU
  if (s) {
    for (void* p : {(void*)D, (void*)Bd, (void*)sl, (void*)sh, (void*)F})
      if (p) cudaFreeAsync(p, s);
    cudaStreamSynchronize(s);
    cudaStreamDestroy(s);
  }
  if (st != DT_OK) {
    free_desc(dd);
    return st;
  }
  Form f;
  f.nb_dev = nb;
  f.bd0_dev = Dv[0] + d0;
  f.bl0_dev = h.bl0;
  f.mono_dev = h.not_mono ? 0 : 1;
  f.tsize_cache = tot[0];
  f.gran_cache = std::min<int64_t>(16, lowp2(h.orr));
  f.lvl_gran_cache = 16;
  f.fits32_cache = (h.lo >= INT32_MIN && h.hi <= INT32_MAX) ? 1 : 0;
  f.sdesc_ok_cache = h.not_sdesc ? 0 : 1;
  f.span_lo = h.lo;
  f.span_hi = h.hi;
  f.span_local_cache = nb < 32 ? 1 : (h.span_good * 2 >= 64 ? 1 : 0);
  if (nb <= 4096) {  // a short merged list: keep the host arrays (the ordinary form)
    f.bd.resize((size_t)nb);
    f.bl.resize((size_t)nb);
    if (cudaMemcpy(f.bd.data(), dd.bd, sizeof(int64_t) * nb, cudaMemcpyDeviceToHost) != cudaSuccess ||
        cudaMemcpy(f.bl.data(), dd.bl, sizeof(int64_t) * nb, cudaMemcpyDeviceToHost) != cudaSuccess) {
      free_desc(dd);
      set_error("GPU flattening: download of a short list failed");
      return DT_ERR_CUDA;
    }
    f.nb_dev = -1;
  }
  const char* no = getenv("DT_NO_SDESC");
  if (h.not_sdesc || nb < 2 || (no && *no && *no != '0')) {
    cudaFree(dd.sdesc);
    cudaFree(dd.wbase);
    dd.sdesc = nullptr;
    dd.wbase = nullptr;
    dd.sdesc_state = 0;
  } else {
    dd.sdesc_state = 1;
  }
  {
    std::lock_guard<std::mutex> g(t->mu);
    t->devs.push_back(dd);
  }
  install_form(t, std::move(f));
  if (getenv("DT_PIPE_DEBUG")) fprintf(stderr, "[dt] GPU flattening: %lld entries -> %lld blocks\n", (long long)n, (long long)nb);
  return DT_OK;
}

// f2: the host arrays of a device-flattened form, downloaded once on demand (host
// consumers: overlap proofs that the device facts do not settle, partial-range launch
// plans, dt_flatten, serialization, another device's upload)
dt_status materialize_host(const Form& f, const DeviceDesc& dd) {
  static std::mutex mm;
  std::lock_guard<std::mutex> g(mm);
  if (!f.host_missing()) return DT_OK;
  Form& F = const_cast<Form&>(f);  // (the form object is owned non-const by its type)
  int cur = -1;
  CU(cudaGetDevice(&cur));
  if (dd.device != cur) CU(cudaSetDevice(dd.device));
  std::vector<int64_t> bd, bl;
  huge_reserve(bd, (size_t)f.nb_dev);
  huge_reserve(bl, (size_t)f.nb_dev);
  bd.resize((size_t)f.nb_dev);
  bl.resize((size_t)f.nb_dev);
  cudaError_t e1 = cudaMemcpy(bd.data(), dd.bd, sizeof(int64_t) * f.nb_dev, cudaMemcpyDeviceToHost);
  cudaError_t e2 = cudaMemcpy(bl.data(), dd.bl, sizeof(int64_t) * f.nb_dev, cudaMemcpyDeviceToHost);
  if (dd.device != cur) cudaSetDevice(cur);
  if (e1 != cudaSuccess || e2 != cudaSuccess) {
    set_error("materialize_host: %s", cudaGetErrorString(e1 != cudaSuccess ? e1 : e2));
    return DT_ERR_CUDA;
  }
  F.bd.swap(bd);
  F.bl.swap(bl);
  F.nb_dev = -1;
  return DT_OK;
}

static dt_status materialize_t(dt_type_s* t, const Form& f) {
  if (!f.host_missing()) return DT_OK;
  if (t->devs.empty()) {
    set_error("device-flattened form without a device descriptor");
    return DT_ERR_ARG;
  }
  return materialize_host(f, t->devs[0]);
}

// f2: the first whole-stream pack of a huge block list (an hindexed list of a
// contiguous element with per-entry lengths, >= DT_PIPE_MIN entries) flattens, uploads
// and packs it in a pipeline -- the paper's T-d2d-pipeline, DEV preparation overlapped
// with the pack kernels ([L18:c1121]-[L18:c1649 §3.2], "almost doubling" uncached,
// [L24:c2562 §5.1]).  A host thread flattens (merges adjacent entries) chunk by chunk into
// the form's arrays; the calling thread uploads each finished run of blocks, scans its
// lengths on the device with the host-known carry, and launches the block-window pack of
// exactly that stream range on the caller's stream (waiting on the upload's event).  A
// chunk's last block stays open until the next chunk (it may still merge).  At the end
// the form and the device descriptor are installed as if committed normally.
static int64_t pipe_min() {
  const char* e = getenv("DT_PIPE_MIN");
  return e ? atoll(e) : (int64_t(1) << 20);
}

static dt_status pipelined_first_pack(dt_type_s* t, int64_t d0, int64_t l0, const void* nc, void* c,
                                      cudaStream_t s) {
  const std::vector<int64_t>& B = t->bls;
  const std::vector<int64_t>& Dv = *t->hdps;
  const size_t n = B.size();
  const char* ce = getenv("DT_PIPE_CHUNK");
  const size_t chunk = ce && atoll(ce) > 0 ? (size_t)atoll(ce) : (size_t(1) << 21);
  int dev = 0;
  CU(cudaGetDevice(&dev));
  Form f;
  huge_reserve(f.bd, n);
  huge_reserve(f.bl, n);
  const int64_t* BD = f.bd.data();  // stable: the capacity covers every merged block
  const int64_t* BL = f.bl.data();
  DeviceDesc dd;
  dd.device = dev;
  cudaStream_t up = nullptr;
  cudaEvent_t ev[2] = {nullptr, nullptr};
  int64_t* sums = nullptr;
  const size_t maxtile = (std::max(chunk, size_t(1) << 20) * 2 + kScanTile - 1) / kScanTile + 1;
  auto fail = [&](cudaError_t e, const char* what) {
    set_error("pipelined first pack: %s: %s", what, cudaGetErrorString(e));
    return DT_ERR_CUDA;
  };
#define PU(call)                                 \
  do {                                           \
    cudaError_t _e = (call);                     \
    if (_e != cudaSuccess) { st = fail(_e, #call); goto out; } \
  } while (0)
  std::atomic<size_t> published{0};
  std::atomic<bool> done{false};
  std::thread producer;
  dt_status st = DT_OK;
  size_t upto = 0;
  int64_t carry = 0, s0 = 0;  // lengths of the uploaded blocks; stream bytes packed so far
  uint64_t orr = 0;
  int launches = 0;
  // the facts later launches ask of the form (granularity, 32-bit template, compact span
  // descriptors) are gathered in the same pass instead of three more passes afterwards
  uint64_t p_or = 0;
  int64_t p_lo = INT64_MAX, p_hi = INT64_MIN;
  bool p_sdesc = true;
  PU(cudaMalloc(&dd.bd, sizeof(int64_t) * n));
  PU(cudaMalloc(&dd.bl, sizeof(int64_t) * n));
  PU(cudaMalloc(&dd.boff, sizeof(int64_t) * n));
  PU(cudaMalloc(&sums, sizeof(int64_t) * maxtile));
  PU(cudaStreamCreateWithFlags(&up, cudaStreamNonBlocking));
  PU(cudaEventCreateWithFlags(&ev[0], cudaEventDisableTiming));
  PU(cudaEventCreateWithFlags(&ev[1], cudaEventDisableTiming));
  producer = std::thread([&] {
    for (size_t i0 = 0; i0 < n; i0 += chunk) {
      const size_t i1 = std::min(n, i0 + chunk);
      for (size_t i = i0; i < i1; i++) {
        const int64_t l = B[i] * l0;
        if (l == 0) continue;
        const int64_t d = Dv[i] + d0;
        if (!f.bd.empty() && f.bd.back() + f.bl.back() == d) {
          f.bl.back() += l;
        } else {
          const size_t w = f.bd.size();
          const int64_t r = d - (w & 31 ? f.bd[w & ~size_t(31)] : d);
          p_sdesc = p_sdesc && r >= INT32_MIN && r <= INT32_MAX;
          p_or |= (uint64_t)d;
          p_lo = std::min(p_lo, d);
          f.bd.push_back(d);
          f.bl.push_back(l);
        }
      }
      const size_t w = f.bd.size();
      published.store(w > 0 ? w - 1 : 0, std::memory_order_release);  // the last block may still grow
    }
    for (size_t i = 0; i < f.bd.size(); i++) {  // merged lengths are final now
      p_or |= (uint64_t)f.bl[i];
      p_hi = std::max(p_hi, f.bd[i] + f.bl[i]);
      p_sdesc = p_sdesc && f.bl[i] < (int64_t(1) << 32);
    }
    published.store(f.bd.size(), std::memory_order_release);
    done.store(true, std::memory_order_release);
  });
  while (true) {
    const bool fin = done.load(std::memory_order_acquire);
    const size_t pub = published.load(std::memory_order_acquire);
    if (pub == upto) {
      if (fin) break;
      std::this_thread::sleep_for(std::chrono::microseconds(20));
      continue;
    }
    if (!fin && pub - upto < chunk / 2) {  // wait for a worthwhile batch
      std::this_thread::sleep_for(std::chrono::microseconds(20));
      continue;
    }
    const size_t m = pub - upto;
    int64_t bsum = 0;
    for (size_t i = upto; i < pub; i++) {
      bsum += BL[i];
      orr |= (uint64_t)BD[i] | (uint64_t)BL[i];  // (cumulative: a batch may start inside an earlier block)
    }
    // this batch packs stream bytes [s0, s1): s1 16-byte aligned (the block-window kernel
    // stores 16-byte vectors), the last batch ends the stream
    const int64_t s1 = fin ? carry + bsum : ((carry + bsum) & ~int64_t(15));  // (fin: pub is the final count)
    const int64_t blen = s1 - s0;
    PU(cudaMemcpyAsync(dd.bd + upto, BD + upto, sizeof(int64_t) * m, cudaMemcpyHostToDevice, up));
    PU(cudaMemcpyAsync(dd.bl + upto, BL + upto, sizeof(int64_t) * m, cudaMemcpyHostToDevice, up));
    {
      const int64_t nt = ((int64_t)m + kScanTile - 1) / kScanTile;
      k_scan_local<<<(unsigned)nt, kScanNT, 0, up>>>(dd.bl + upto, dd.boff + upto, sums, (int64_t)m);
      k_scan_sums<<<1, kScanNT, 0, up>>>(sums, nt, carry);  // carry: lengths of the blocks before `upto`
      k_scan_add<<<(unsigned)nt, kScanNT, 0, up>>>(dd.boff + upto, sums, (int64_t)m);
      PU(cudaGetLastError());
    }
    PU(cudaEventRecord(ev[launches & 1], up));
    PU(cudaStreamWaitEvent(s, ev[launches & 1], 0));
    {
      // block-window pack of stream bytes [carry, carry + blen): blocks [0, pub) are valid
      KP P;
      std::memset(&P, 0, sizeof(P));
      P.nc = (const uint8_t*)nc;
      P.c = (uint8_t*)c + s0;
      P.pos = s0;
      P.len = blen;
      P.tsize = t->size;
      P.nblocks = (int64_t)pub;
      P.bd = dd.bd;
      P.bl = dd.bl;
      P.boff = dd.boff;
      P.nlev = 0;
      P.ftsize = make_fd((uint64_t)P.tsize);
      P.fnb = make_fd((uint64_t)P.nblocks);
      const int64_t g =
          lowp2(orr | (uint64_t)(uintptr_t)nc | (uint64_t)(uintptr_t)c | (uint64_t)s0 | (uint64_t)blen);
      const int sms = num_sms();
      const int64_t max_warps = (int64_t)sms * 4 * 8;
      int64_t nw = std::min<int64_t>(max_warps, std::max<int64_t>(1, (blen + 4095) / 4096));
      int64_t per = (blen + nw - 1) / nw;
      per = (per + kBlkWin - 1) / kBlkWin * kBlkWin;
      nw = (blen + per - 1) / per;
      P.per_warp = per;
      const unsigned grid = (unsigned)((nw + 7) / 8);
      const size_t smem = 8 * (kBlkWin / g) * sizeof(int64_t);
      if (blen > 0) switch (g) {
        case 1: k_blk<false, 1><<<grid, 256, smem, s>>>(P); break;
        case 2: k_blk<false, 2><<<grid, 256, smem, s>>>(P); break;
        case 4: k_blk<false, 4><<<grid, 256, smem, s>>>(P); break;
        case 8: k_blk<false, 8><<<grid, 256, smem, s>>>(P); break;
        default: k_blk<false, 16><<<grid, 256, smem, s>>>(P); break;
      }
      PU(cudaGetLastError());
    }
    PU(cudaStreamSynchronize(up));  // (sums is reused by the next batch)
    carry += bsum;
    s0 = s1;
    upto = pub;
    launches++;
  }
  if (carry != t->size || s0 != t->size) {
    set_error("pipelined first pack: %lld of %lld bytes", (long long)s0, (long long)t->size);
    st = DT_ERR_ARG;
    goto out;
  }
out:
  if (producer.joinable()) producer.join();
#undef PU
  if (sums) cudaFree(sums);
  if (up) cudaStreamDestroy(up);
  for (auto e : ev)
    if (e) cudaEventDestroy(e);
  if (st != DT_OK) {
    free_desc(dd);
    return st;
  }
  if (getenv("DT_PIPE_DEBUG")) fprintf(stderr, "[dt] pipelined first pack: %zu blocks, %d batches\n", f.bd.size(), launches);
  f.gran_cache = std::min<int64_t>(16, lowp2(p_or));
  f.fits32_cache = (p_lo >= INT32_MIN && p_hi <= INT32_MAX) ? 1 : 0;
  f.sdesc_ok_cache = p_sdesc ? 1 : 0;
  {
    std::lock_guard<std::mutex> g(t->mu);
    t->devs.push_back(dd);
    t->lazy_pipe = false;
  }
  install_form(t, std::move(f));
  return DT_OK;
}

static dt_status pack_common(bool unpack, dt_t t, int64_t count, const void* nc, void* c, int64_t pos, int64_t* len,
                             void* stream, bool check_ptrs = true) {
  if (!t || !len || count < 0 || pos < 0 || *len < 0) {
    set_error("dt_%s: bad argument", unpack ? "unpack" : "pack");
    return DT_ERR_ARG;
  }
  if (!t->committed) {
    set_error("dt_%s: type not committed", unpack ? "unpack" : "pack");
    return DT_ERR_NOT_COMMITTED;
  }
  const int64_t total = count * t->size;
  int64_t n = pos >= total ? 0 : std::min<int64_t>(*len, total - pos);
  *len = n;
  if (n == 0) return DT_OK;
  if (!nc || !c) {
    set_error("dt_%s: NULL buffer", unpack ? "unpack" : "pack");
    return DT_ERR_ARG;
  }
  if (g_check_ptrs && check_ptrs) {
    dt_status st = check_dev_ptr((const uint8_t*)nc + t->true_lb, "origin");
    if (st != DT_OK) return st;
    st = check_dev_ptr(c, "packed");
    if (st != DT_OK) return st;
  }
  if (t->lazy_pipe) {  // f2: the first whole-stream pack of a huge block list, pipelined
    int64_t d0 = 0, l0 = 0;
    if (!unpack && count == 1 && pos == 0 && n == t->size && pipe_list(t, &d0, &l0))
      return pipelined_first_pack(t, d0, l0, nc, c, (cudaStream_t)stream);
    t->lazy_pipe = false;  // any other first use flattens and uploads as usual
  }
  DeviceDesc* dd = nullptr;
  dt_status st = ensure_committed_on_device(t, &dd);
  if (st != DT_OK) return st;
  const Form& f = get_form(t);
  if (unpack) {
    std::lock_guard<std::mutex> g(t->mu);
    if (t->ovl_count != count) {
      t->ovl_result = check_nonoverlap(t, f, count);
      t->ovl_count = count;
    }
    if (t->ovl_result != 1) {
      set_error("dt_unpack: typemap entries overlap%s", t->ovl_result < 0 ? " (could not be proven disjoint)" : "");
      return DT_ERR_OVERLAP;
    }
  }
  return launch_pack_unpack(unpack, t, f, *dd, count, nc, c, pos, n, stream);
}

}  // namespace dt

using namespace dt;

extern "C" {

dt_status dt_commit(dt_t t) {
  if (!t) {
    set_error("dt_commit: NULL type");
    return DT_ERR_ARG;
  }
  {
    // f2: a huge block list is flattened on the GPU (default, DT_FLATTEN=gpu), or by its
    // first whole-stream pack pipelined with it (DT_FLATTEN=pipe: the paper's overlap of
    // host preparation with the kernels), or on the host (DT_FLATTEN=host / DT_NO_PIPE)
    int64_t d0, l0;
    const char* fm = getenv("DT_FLATTEN");
    const std::string mode = getenv("DT_NO_PIPE") ? "host" : fm ? fm : "gpu";
    if (!t->committed && !t->form && t->kind == K_HINDEXED && t->count >= pipe_min() && mode != "host" &&
        pipe_list(t, &d0, &l0)) {
      if (mode == "pipe") {
        t->lazy_pipe = true;
        t->committed = true;
        if (const char* e = getenv("DT_NOCHECK")) g_check_ptrs = (e[0] == '0');
        return DT_OK;
      }
      bool fallback = false;
      dt_status gs = gpu_flatten(t, d0, l0, &fallback);
      if (gs == DT_OK) {
        t->committed = true;
        if (const char* e = getenv("DT_NOCHECK")) g_check_ptrs = (e[0] == '0');
        return DT_OK;
      }
      if (!fallback) return gs;  // (entries of count 0: the host flattening below)
    }
  }
  try {
    get_form(t);
  } catch (...) {
    set_error("dt_commit: flattening failed (too many blocks or out of memory)");
    return DT_ERR_NOMEM;
  }
  DeviceDesc* dd = nullptr;
  dt_status st = ensure_committed_on_device(t, &dd);
  if (st != DT_OK) return st;
  t->committed = true;
  if (const char* e = getenv("DT_NOCHECK")) g_check_ptrs = (e[0] == '0');
  return DT_OK;
}

dt_status dt_pack(dt_t t, int64_t count, const void* origin, void* packed, int64_t pos, int64_t* len, void* stream) {
  return pack_common(false, t, count, origin, packed, pos, len, stream);
}

dt_status dt_unpack(dt_t t, int64_t count, const void* packed, void* origin, int64_t pos, int64_t* len,
                    void* stream) {
  return pack_common(true, t, count, origin, const_cast<void*>(packed), pos, len, stream);
}

// f1: fused datatype -> datatype copy on the current device (no packed buffer).
static dt_status make_kp(dt_type_s* t, int64_t count, const void* nc, int64_t n, KP& P, const Form** fo,
                         DeviceDesc** ddo) {
  DeviceDesc* dd = nullptr;
  dt_status st = ensure_committed_on_device(t, &dd);
  if (st != DT_OK) return st;
  const Form& f = get_form(t);
  KLevels L;
  build_levels(f, dd, t, count, L);
  std::memset(&P, 0, sizeof(P));
  P.nc = (const uint8_t*)nc;
  P.pos = 0;
  P.len = n;
  P.tsize = f.tsize();
  P.nblocks = f.nblocks();
  P.bd = dd->bd;
  P.bl = dd->bl;
  P.boff = dd->boff;
  P.bd0 = f.first_bd();
  P.bl0 = f.first_bl();
  P.nlev = L.n;
  for (int i = 0; i < L.n; i++) {
    P.cnt[i] = L.cnt[i];
    P.stride[i] = L.stride[i];
    P.table[i] = L.table[i];
    P.fcnt[i] = make_fd((uint64_t)L.cnt[i]);
  }
  P.ftsize = make_fd((uint64_t)P.tsize);
  *fo = &f;
  *ddo = dd;
  return DT_OK;
}

}  // extern "C"

// receive-side legality: the destination typemap must not overlap (cached per count)
int dt::nonoverlap_cached(dt_type_s* rt, int64_t rcount) {
  const Form& fr = get_form(rt);
  std::lock_guard<std::mutex> g(rt->mu);
  if (rt->ovl_count != rcount) {
    rt->ovl_result = check_nonoverlap(rt, fr, rcount);
    rt->ovl_count = rcount;
  }
  return rt->ovl_result;
}

// Parameters of a fused type -> type copy of n stream bytes from (st, scount, src)
// to (rt, rcount, dst) and its kernel family, as dt_copy launches it: 1 dual block
// walk (long runs), 2 dual word tables, 4 smem-staged (cp.async gather by the
// source layout, scatter by the destination layout).  Word tables are attached.
dt_status dt::dual_params(dt_type_s* st, int64_t scount, const void* src, dt_type_s* rt, int64_t rcount, void* dst,
                      int64_t n, KP& S, KP& R, int* kind, int64_t* gran) {
  const Form *fs, *fr;
  DeviceDesc *ds, *dr;
  dt_status s1 = make_kp(st, scount, src, n, S, &fs, &ds);
  if (s1 != DT_OK) return s1;
  s1 = make_kp(rt, rcount, dst, n, R, &fr, &dr);
  if (s1 != DT_OK) return s1;
  KLevels Ls, Lr;
  build_levels(*fs, ds, st, scount, Ls);
  build_levels(*fr, dr, rt, rcount, Lr);
  int64_t gs = 1, gr = 1;
  plan_kernel(*fs, Ls, (uint64_t)(uintptr_t)src, 0, 0, n, &gs);
  plan_kernel(*fr, Lr, (uint64_t)(uintptr_t)dst, 0, 0, n, &gr);
  const int64_t g = std::min(gs, gr);
  const double ms = (double)S.tsize / (double)S.nblocks, mr = (double)R.tsize / (double)R.nblocks;
  const bool words_ok = S.tsize % g == 0 && R.tsize % g == 0 && (S.tsize + R.tsize) / g <= kMaxWordTable &&
                        template_fits_int32(*fs) && template_fits_int32(*fr);
  const char* fk = getenv("DT_FORCE_KERNEL");
  const int force = fk ? atoi(fk) : 0;
  const double mm = std::min(ms, mr);
  const bool use_words = words_ok && force != 1 && (force == 2 || mm < 256.0 || (g == 16 && mm < 1024.0));
  *gran = g;
  if (!use_words) {
    *kind = 1;
    return DT_OK;
  }
  const int32_t *wa = nullptr, *wb = nullptr;
  s1 = ensure_wtab(*fs, *ds, g, &wa);
  if (s1 != DT_OK) return s1;
  s1 = ensure_wtab(*fr, *dr, g, &wb);
  if (s1 != DT_OK) return s1;
  S.wtab = wa;
  S.nwords = (int32_t)(S.tsize / g);
  R.wtab = wb;
  R.nwords = (int32_t)(R.tsize / g);
  // staged for >= 8-byte words (DT_FORCE_KERNEL=2 keeps the register word kernel)
  *kind = (g >= stage_min_g() && g >= 4 && force != 2) ? 4 : 2;
  return DT_OK;
}

extern "C" {

static dt_status copy_typed(dt_t st, int64_t scount, const void* src, dt_t rt, int64_t rcount, void* dst,
                            void* stream) {
  if (!st || !rt || scount < 0 || rcount < 0) {
    set_error("dt_copy: bad argument");
    return DT_ERR_ARG;
  }
  if (!st->committed || !rt->committed) {
    set_error("dt_copy: type not committed");
    return DT_ERR_NOT_COMMITTED;
  }
  const int64_t n = scount * st->size;
  if (n > rcount * rt->size) {
    set_error("dt_copy: %lld bytes do not fit a %lld-byte receive layout", (long long)n,
              (long long)(rcount * rt->size));
    return DT_ERR_TRUNCATE;
  }
  if (n == 0) return DT_OK;
  if (!src || !dst) {
    set_error("dt_copy: NULL buffer");
    return DT_ERR_ARG;
  }
  if (g_check_ptrs) {
    dt_status s1 = check_dev_ptr((const uint8_t*)src + st->true_lb, "source");
    if (s1 != DT_OK) return s1;
    s1 = check_dev_ptr((const uint8_t*)dst + rt->true_lb, "destination");
    if (s1 != DT_OK) return s1;
  }
  if (nonoverlap_cached(rt, rcount) != 1) {
    set_error("dt_copy: destination typemap entries overlap");
    return DT_ERR_OVERLAP;
  }
  KP S, R;
  int kind = 1;
  int64_t g = 1;
  dt_status s1 = dual_params(st, scount, src, rt, rcount, dst, n, S, R, &kind, &g);
  if (s1 != DT_OK) return s1;
  cudaStream_t s = (cudaStream_t)stream;
  const int sms = num_sms();
  if (kind == 4) {  // staged: cp.async gathers by S into smem tiles, scatter by R
    const size_t smem2 = (size_t)kStageBufs * kStageTile + sizeof(int32_t) * (size_t)(S.nwords + R.nwords);
    bool& attr = devl().dual_attr;
    if (!attr) {
      cudaFuncSetAttribute(k_dual_stage<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 * 1024);
      cudaFuncSetAttribute(k_dual_stage<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 * 1024);
      cudaFuncSetAttribute(k_dual_stage<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 * 1024);
      attr = true;
    }
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_dual_stage<16>, 256, smem2) != cudaSuccess || occ < 1)
      occ = 1;
    const int64_t ntiles = (n + kStageTile - 1) / kStageTile;
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * occ, ntiles));
    if (g == 4) k_dual_stage<4><<<grid, 256, smem2, s>>>(S, R, n, ntiles);
    else if (g == 8) k_dual_stage<8><<<grid, 256, smem2, s>>>(S, R, n, ntiles);
    else k_dual_stage<16><<<grid, 256, smem2, s>>>(S, R, n, ntiles);
  } else if (kind == 2) {
    const size_t smem = sizeof(int32_t) * (size_t)(S.nwords + R.nwords);
    const int64_t nwords = n / g;
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * 6, (nwords + 1023) / 1024));
    switch (g) {
      case 1: k_dual_word<1><<<grid, 256, smem, s>>>(S, R, n); break;
      case 2: k_dual_word<2><<<grid, 256, smem, s>>>(S, R, n); break;
      case 4: k_dual_word<4><<<grid, 256, smem, s>>>(S, R, n); break;
      case 8: k_dual_word<8><<<grid, 256, smem, s>>>(S, R, n); break;
      default: k_dual_word<16><<<grid, 256, smem, s>>>(S, R, n); break;
    }
  } else {
    const int64_t nw = std::min<int64_t>((int64_t)sms * 3 * 8, std::max<int64_t>(1, (n + 4095) / 4096));
    int64_t per = (n + nw - 1) / nw;
    per = (per + 511) & ~int64_t(511);
    const int64_t nwr = (n + per - 1) / per;
    k_dual_seg<<<(unsigned)((nwr + 7) / 8), 256, 0, s>>>(S, R, n, per);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(e, "dt_copy launch");
  return DT_OK;
}

dt_status dt_copy(dt_t st, int64_t scount, const void* src, dt_t rt, int64_t rcount, void* dst, void* stream) {
  return copy_typed(st, scount, src, rt, rcount, dst, stream);
}

dt_status dt_plan(dt_t t, int64_t count, uint64_t origin_addr, uint64_t packed_addr, int64_t pos, int64_t len,
                  int* kernel, int64_t* granularity) {
  if (!t || !kernel || !granularity || count < 0 || pos < 0 || len < 0) {
    set_error("dt_plan: bad argument");
    return DT_ERR_ARG;
  }
  const Form* f;
  try {
    f = &get_form(t);
  } catch (...) {
    set_error("dt_plan: flattening failed");
    return DT_ERR_NOMEM;
  }
  const int64_t total = count * t->size;
  const int64_t n = pos >= total ? 0 : std::min<int64_t>(len, total - pos);
  Eff E = effective(*f, nullptr, t, count);
  *granularity = 1;
  *kernel = n <= 0 ? 0 : E.merged ? 1 : plan_kernel(*f, E.L, origin_addr, packed_addr, pos, n, granularity);
  return DT_OK;
}

// Host-buffer entry points: stage the span the layout touches through device
// scratch memory (H2D), run the GPU kernel, copy the result back (D2H).
static void* g_scratch[2] = {nullptr, nullptr};
static size_t g_scratch_sz[2] = {0, 0};
static int g_scratch_dev = -1;
static std::mutex g_scratch_mu;

static dt_status scratch(int i, size_t n, void** out) {
  int dev = 0;
  CU(cudaGetDevice(&dev));
  if (g_scratch_dev != dev) {
    for (int k = 0; k < 2; k++) { g_scratch[k] = nullptr; g_scratch_sz[k] = 0; }
    g_scratch_dev = dev;
  }
  if (g_scratch_sz[i] < n) {
    if (g_scratch[i]) cudaFree(g_scratch[i]);
    g_scratch[i] = nullptr;
    g_scratch_sz[i] = 0;
    CU(cudaMalloc(&g_scratch[i], n));
    g_scratch_sz[i] = n;
  }
  *out = g_scratch[i];
  return DT_OK;
}

// Host-link pipeline for pinned buffers: the SMs move the layout side over the host link
// (zero-copy gather from / scatter to the pinned origin, into / out of a device ring of
// chunks) while the copy engine moves the packed side chunk by chunk in the other
// direction -- the paper's pipelining of pack with the transfer ([L18:c4394 §4.1]) applied
// to the host link.  Measured on B200 (tools/micro/zerocopy.cu): a kernel that reads and
// writes host memory at once tops out at ~74-79 GB/s, a zero-copy read (51 GB/s) or write
// (52 GB/s) next to a copy-engine copy the other way is not capped that way (two memcpys:
// 99 GB/s).  Chunk C = DT_HOST_CHUNK (default 4 MiB), 3 ring slots; DT_HOST_PIPE=0 keeps the
// single zero-copy kernel for both directions.  Ordered after the caller's stream; synchronous like the rest of
// the host entry points.
struct HostPipe {
  int dev = -1;
  cudaStream_t ks = nullptr, cs = nullptr;
  cudaEvent_t ev_start = nullptr, ev_k[3] = {}, ev_c[3] = {}, ev_end[2] = {};
};
static HostPipe g_hp;

static dt_status host_pipe(bool unpack, dt_t t, int64_t count, uint8_t* dorig, uint8_t* hpk, int64_t pos, int64_t n,
                           cudaStream_t us) {
  constexpr int D = 3;
  const int64_t C = getenv("DT_HOST_CHUNK") ? std::max<int64_t>(4096, atoll(getenv("DT_HOST_CHUNK")) & ~int64_t(4095))
                                                   : (int64_t)4 << 20;
  int dev = 0;
  CU(cudaGetDevice(&dev));
  if (g_hp.dev != dev) {
    CU(cudaStreamCreateWithFlags(&g_hp.ks, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&g_hp.cs, cudaStreamNonBlocking));
    CU(cudaEventCreateWithFlags(&g_hp.ev_start, cudaEventDisableTiming));
    for (int i = 0; i < D; i++) {
      CU(cudaEventCreateWithFlags(&g_hp.ev_k[i], cudaEventDisableTiming));
      CU(cudaEventCreateWithFlags(&g_hp.ev_c[i], cudaEventDisableTiming));
    }
    for (int i = 0; i < 2; i++) CU(cudaEventCreateWithFlags(&g_hp.ev_end[i], cudaEventDisableTiming));
    g_hp.dev = dev;
  }
  void* ring = nullptr;
  dt_status st = scratch(1, (size_t)(D * C), &ring);
  if (st != DT_OK) return st;
  uint8_t* rb = (uint8_t*)ring;
  const cudaStream_t ks = g_hp.ks, cs = g_hp.cs;
  CU(cudaEventRecord(g_hp.ev_start, us));
  CU(cudaStreamWaitEvent(ks, g_hp.ev_start, 0));
  CU(cudaStreamWaitEvent(cs, g_hp.ev_start, 0));
  const int64_t nk = (n + C - 1) / C;
  for (int64_t k = 0; k < nk; k++) {
    const int slot = (int)(k % D);
    int64_t m = std::min(C, n - k * C);
    uint8_t* sl = rb + (size_t)slot * C;
    if (!unpack) {
      if (k >= D) CU(cudaStreamWaitEvent(ks, g_hp.ev_c[slot], 0));  // slot's previous D2H done
      st = pack_common(false, t, count, dorig, sl, pos + k * C, &m, ks, /*check_ptrs=*/false);
      if (st != DT_OK) return st;
      CU(cudaEventRecord(g_hp.ev_k[slot], ks));
      CU(cudaStreamWaitEvent(cs, g_hp.ev_k[slot], 0));
      CU(cudaMemcpyAsync(hpk + k * C, sl, (size_t)m, cudaMemcpyDeviceToHost, cs));
      CU(cudaEventRecord(g_hp.ev_c[slot], cs));
    } else {
      if (k >= D) CU(cudaStreamWaitEvent(cs, g_hp.ev_k[slot], 0));  // slot's previous unpack done
      CU(cudaMemcpyAsync(sl, hpk + k * C, (size_t)m, cudaMemcpyHostToDevice, cs));
      CU(cudaEventRecord(g_hp.ev_c[slot], cs));
      CU(cudaStreamWaitEvent(ks, g_hp.ev_c[slot], 0));
      st = pack_common(true, t, count, dorig, sl, pos + k * C, &m, ks, /*check_ptrs=*/false);
      if (st != DT_OK) return st;
      CU(cudaEventRecord(g_hp.ev_k[slot], ks));
    }
  }
  CU(cudaEventRecord(g_hp.ev_end[0], ks));
  CU(cudaEventRecord(g_hp.ev_end[1], cs));
  CU(cudaStreamWaitEvent(us, g_hp.ev_end[0], 0));
  CU(cudaStreamWaitEvent(us, g_hp.ev_end[1], 0));
  CU(cudaStreamSynchronize(us));
  return DT_OK;
}

static dt_status host_common(bool unpack, dt_t t, int64_t count, const void* a, void* b, int64_t pos, int64_t* len,
                             void* stream) {
  if (!t || !len || count < 0 || pos < 0 || *len < 0 || !a || !b) {
    set_error("dt_%s_host: bad argument", unpack ? "unpack" : "pack");
    return DT_ERR_ARG;
  }
  if (!t->committed) {
    set_error("dt_%s_host: type not committed", unpack ? "unpack" : "pack");
    return DT_ERR_NOT_COMMITTED;
  }
  const int64_t total = count * t->size;
  const int64_t n = pos >= total ? 0 : std::min<int64_t>(*len, total - pos);
  *len = n;
  if (n == 0) return DT_OK;
  // span of count instances: [true_lb + min(0,(count-1)ext), true_ub + max(0,(count-1)ext))
  const int64_t last = (count - 1) * t->extent();
  const int64_t lo = t->true_lb + std::min<int64_t>(0, last);
  const int64_t hi = t->true_ub + std::max<int64_t>(0, last);
  // Pinned (page-locked, device-mapped) host buffers: the pack/unpack kernel itself reads
  // and writes host memory over the host link (zero-copy) -- only the typemap's bytes and
  // the packed stream cross it, no span staging and no extra pass.  Pageable buffers are
  // staged through device scratch below.
  {
    const uint8_t* nc = unpack ? (const uint8_t*)b : (const uint8_t*)a;
    const uint8_t* pk = unpack ? (const uint8_t*)a : (const uint8_t*)b;
    void *d0 = nullptr, *d1 = nullptr, *d2 = nullptr;
    if (!getenv("DT_HOST_STAGED") && host_mapped(nc + lo, &d0) && host_mapped(nc + hi - 1, &d1) &&
        host_mapped(pk, &d2) && (uint8_t*)d1 - (uint8_t*)d0 == hi - lo - 1) {
      uint8_t* dorig = (uint8_t*)d0 - lo;
      // pipeline: unpack only by default (CE H2D of packed chunks + zero-copy scatter: C2
      // 1.88 -> 1.71 ms); for pack the SM's zero-copy reads slow down next to the CE's D2H
      // (1.87 -> 2.21 ms), so pack keeps the single kernel (DT_HOST_PIPE=2 pipelines both)
      const char* hp = getenv("DT_HOST_PIPE");
      const int mode = hp ? atoi(hp) : 1;
      if (n > ((int64_t)8 << 20) && (mode == 2 || (mode == 1 && unpack))) {
        std::lock_guard<std::mutex> g(g_scratch_mu);
        return host_pipe(unpack, t, count, dorig, (uint8_t*)pk, pos, n, (cudaStream_t)stream);
      }
      int64_t m = n;
      dt_status st = pack_common(unpack, t, count, dorig, d2, pos, &m, stream, /*check_ptrs=*/false);
      if (st != DT_OK) return st;
      CU(cudaStreamSynchronize((cudaStream_t)stream));
      return DT_OK;
    }
  }
  std::lock_guard<std::mutex> g(g_scratch_mu);
  void *dspan, *dpack;
  dt_status st = scratch(0, (size_t)(hi - lo), &dspan);
  if (st != DT_OK) return st;
  st = scratch(1, (size_t)n, &dpack);
  if (st != DT_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  uint8_t* dorigin = (uint8_t*)dspan - lo;
  int64_t m = n;
  if (!unpack) {
    const uint8_t* horigin = (const uint8_t*)a;
    CU(cudaMemcpyAsync(dspan, horigin + lo, (size_t)(hi - lo), cudaMemcpyHostToDevice, s));
    st = pack_common(false, t, count, dorigin, dpack, pos, &m, stream, false);
    if (st == DT_OK) CU(cudaMemcpyAsync(b, dpack, (size_t)n, cudaMemcpyDeviceToHost, s));
  } else {
    uint8_t* horigin = (uint8_t*)b;
    // gaps must stay untouched: bring the destination span in, scatter, send it back
    CU(cudaMemcpyAsync(dspan, horigin + lo, (size_t)(hi - lo), cudaMemcpyHostToDevice, s));
    CU(cudaMemcpyAsync(dpack, a, (size_t)n, cudaMemcpyHostToDevice, s));
    st = pack_common(true, t, count, dorigin, dpack, pos, &m, stream, false);
    if (st == DT_OK) CU(cudaMemcpyAsync(horigin + lo, dspan, (size_t)(hi - lo), cudaMemcpyDeviceToHost, s));
  }
  if (st != DT_OK) return st;
  CU(cudaStreamSynchronize(s));
  return DT_OK;
}

dt_status dt_pack_host(dt_t t, int64_t count, const void* origin, void* packed, int64_t pos, int64_t* len,
                       void* stream) {
  return host_common(false, t, count, origin, packed, pos, len, stream);
}
dt_status dt_unpack_host(dt_t t, int64_t count, const void* packed, void* origin, int64_t pos, int64_t* len,
                         void* stream) {
  return host_common(true, t, count, packed, origin, pos, len, stream);
}

}  // extern "C"
