// dt_xfer.cu — GPU<->GPU pipelined transfer of non-contiguous data (S7).
//
// Paper ([L18:c4394]-[L20:c4670 §4.1], Fig. 4): the sender packs fragments into a
// GPU staging buffer exposed to the receiver over CUDA IPC; the receiver unpacks
// each fragment as soon as the sender signals it and acknowledges it so the
// fragment can be reused; with a pipeline the cost falls to "the cost of the
// data transfer plus the cost of the most expensive operation (pack or unpack)
// on a single fragment" ([L18:c4932]).  Connection setup exchanges the IPC
// handle once ([L20:c3123], [L20:c3807]); the receiver sends "start packing"
// ([L20:c3973]); the sender signals "unpack fragment i" ([L20:c3380]) and the
// receiver acks ([L20:c4133]).
//
// B200 design:
//  * P2P mode: ONE persistent kernel per call (or per group of calls) whose
//    send-role CTAs pack fragment k straight into the receiver's ring slot k%D in
//    peer HBM over NVLink (remote 16-byte stores), then publish it with a
//    release.sys add of the bytes written to the receiver's ready[slot]; the
//    receive-role CTAs spin (ld.acquire.sys) on their local ready[slot], unpack
//    the slot into the user's layout and add the bytes consumed to the sender's
//    ack[slot].  Chunk != launch: the chunk size only sets flow-control
//    granularity.  Counters are cumulative bytes per slot; each side keeps its
//    base per (peer, channel) in device memory, double-buffered by message parity.
//    Header {seq, nbytes} + "go" word implement the handshake and truncation check.
//  * NCCL mode: double-buffered chunks: pack(k) -> ncclSend/ncclRecv -> unpack(k)
//    on three internal streams with per-slot events.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <unistd.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "dt_device.cuh"
#include "dt_internal.h"

namespace dt {

constexpr int kMaxOps = 16;
constexpr int kMaxCh = 6;   // concurrent messages per (pair, direction) inside one group
constexpr int kMaxSub = 64; // sub-rings (one per sending CTA) per message
constexpr uint64_t kAbort = 1ull << 63;

struct XOp {
  KP P;            // pack (send role) or unpack (recv role) over the user's layout
  int32_t role;    // 0 send, 1 recv
  int32_t kind;    // 1 segment walk, 2 word table, 4 smem/TMA staging, 6 record spans, 7 block spans
  int32_t single;  // segment walk over a single-block template
  int32_t g;       // word granularity
  int64_t n;       // send: bytes; recv: capacity in bytes
  int64_t chunk;
  int32_t depth, cta0, ncta, rep;  // rep (send role): CTAs per sub-ring, alternating fragments
  uint8_t* ring;   // slot 0 of the (pair, channel) ring (send: peer memory; recv: local)
  uint64_t* ready; // [depth]  send: peer; recv: local
  uint64_t* ack;   // [depth]  send: local; recv: peer
  uint64_t* hdr;   // [2] {seq, nbytes}  send: peer; recv: local
  uint64_t* go;    // [1]     send: local; recv: peer
  const uint64_t* base_in;  // [depth] cumulative bytes per slot before this message
  uint64_t* base_out;       // [depth] after it
  uint64_t seq;
  int32_t* err;
  RecGeo rg;       // kind 6: record-span geometry (per-fragment element range set on the device)
};

struct XArgs {
  int32_t nops;
  int32_t wt_off;  // byte offset of the word table in dynamic smem (after the staging buffers)
  int32_t flags;
  int32_t pad2;  // tuning switches (DT_XFER_FLAGS): bit1 = no sleep in polls, bit2 = SC system fence before each flag
  int64_t timeout_ns;
  XOp ops[kMaxOps];
};

// pack or unpack stream bytes [lo, lo+len) of the current chunk with this CTA.
// cb: the slot base such that stream byte x of the message lives at cb + x.  The
// op's parameters stay in the grid-constant bank (no per-fragment struct copy).
template <bool UNPACK>
__device__ __forceinline__ void cta_chunk(const XOp& X, uint8_t* cb, int64_t lo, int64_t len, const int32_t* wt,
                                          uint8_t* sbuf, uint64_t* mbar) {
  const KP& P = X.P;
  const int64_t hi = lo + len;
  constexpr int POL = UNPACK ? LD_CG : LD_CS;  // ring slots are rewritten by the peer: bypass L1
  if (X.kind == 6) {  // record spans: the CTA's warps take RB-record batches of the fragment
    const int64_t hb = hi - len % X.g;  // a ragged tail (< G bytes, last fragment) is walked below
    RecGeo R = X.rg;
    R.e_lo = lo / P.tsize;
    R.e_hi = (hb + P.tsize - 1) / P.tsize;
    R.b0 = R.e_lo & ~int64_t(31);
    R.nbatch = (R.e_hi - R.b0 + R.RB - 1) / R.RB;
    const int nwc = blockDim.x >> 5, w = threadIdx.x >> 5;
    uint8_t* buf = sbuf + w * (R.RB * R.spanB);
    int64_t* sd = reinterpret_cast<int64_t*>(sbuf + nwc * (R.RB * R.spanB)) + w * R.RB;
    uint16_t* omap = reinterpret_cast<uint16_t*>(sbuf + nwc * (R.RB * R.spanB) + nwc * R.RB * 8);
    const int lane = threadIdx.x & 31;
    if (lo < hb) {
      switch (X.g) {
        case 4: rec_range<UNPACK, 4, POL>(P, R, cb, lo, hb, buf, sd, omap, w, nwc, lane); break;
        case 8: rec_range<UNPACK, 8, POL>(P, R, cb, lo, hb, buf, sd, omap, w, nwc, lane); break;
        default: rec_range<UNPACK, 16, POL>(P, R, cb, lo, hb, buf, sd, omap, w, nwc, lane); break;
      }
    }
    if (hb < hi && w == nwc - 1) seg_range<UNPACK, false, POL>(P, cb, hb, hi, lane);
    return;
  }
  if (X.kind == 7) {  // block spans: the CTA's warps take equal 16-byte-multiple slices of the fragment
    const int nwc = blockDim.x >> 5, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t body = len - len % X.g;  // a ragged tail (< G bytes, last fragment) is walked below
    int64_t per = (body + nwc - 1) / nwc;
    per = (per + 15) & ~int64_t(15);
    const int64_t a = lo + (int64_t)w * per, b = min(a + per, lo + body);
    if (a < b) {
      const PlanEnt st = span_start(P, a, lane);
      uint8_t* sm = sbuf + (size_t)w * kSpanWarpSmem;
      switch (X.g) {
        case 4: span_range<UNPACK, 4, POL>(P, cb, st, b, lane, sm); break;
        case 8: span_range<UNPACK, 8, POL>(P, cb, st, b, lane, sm); break;
        default: span_range<UNPACK, 16, POL>(P, cb, st, b, lane, sm); break;
      }
    }
    if (body < len && w == nwc - 1) seg_range<UNPACK, false, POL>(P, cb, lo + body, hi, lane);
    return;
  }
  if (X.kind == 4) {  // smem/TMA staging: bulk store into the (peer) ring slot / bulk load from it
    const int64_t bh = hi - len % X.g;  // words; a ragged tail (< G bytes, last fragment) is walked below
    switch (X.g) {
      case 8:
        if (UNPACK) stage_unpack<8, kXferStageBufs>(P, cb, wt, lo, bh, sbuf, mbar);
        else stage_pack<8, kXferStageBufs>(P, cb, wt, lo, bh, sbuf);
        break;
      default:
        if (UNPACK) stage_unpack<16, kXferStageBufs>(P, cb, wt, lo, bh, sbuf, mbar);
        else stage_pack<16, kXferStageBufs>(P, cb, wt, lo, bh, sbuf);
        break;
    }
    if (bh < hi) {
      __syncthreads();
      if (threadIdx.x < 32) seg_range<UNPACK, false, POL>(P, cb, bh, hi, threadIdx.x & 31);
    }
    return;
  }
  if (X.kind == 2) {
    const int64_t body = len - len % X.g;
    // few CTAs carry the whole transfer: keep 4 vectors per thread in flight (512 threads: 32 KiB/CTA)
    switch (X.g) {
      case 1: word_range<UNPACK, 1, 16, POL, 2>(P, cb, lo, lo + body, wt, threadIdx.x, blockDim.x); break;
      case 2: word_range<UNPACK, 2, 16, POL, 2>(P, cb, lo, lo + body, wt, threadIdx.x, blockDim.x); break;
      case 4: word_range<UNPACK, 4, 16, POL, 4>(P, cb, lo, lo + body, wt, threadIdx.x, blockDim.x); break;
      case 8: word_range<UNPACK, 8, 16, POL, 4>(P, cb, lo, lo + body, wt, threadIdx.x, blockDim.x); break;
      default: word_range<UNPACK, 16, 16, POL, 4>(P, cb, lo, lo + body, wt, threadIdx.x, blockDim.x); break;
    }
    if (body < len && threadIdx.x < 32)  // ragged tail (< G bytes): one warp walks it
      seg_range<UNPACK, false, POL>(P, cb, lo + body, hi, threadIdx.x & 31);
    return;
  }
  const int nw = blockDim.x >> 5, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  int64_t per = (len + nw - 1) / nw;
  per = (per + 127) & ~int64_t(127);
  const int64_t a = lo + (int64_t)w * per, b = min(a + per, hi);
  if (X.single) seg_range<UNPACK, true, POL>(P, cb, a, b, lane);
  else seg_range<UNPACK, false, POL>(P, cb, a, b, lane);
}

constexpr int kXferThreads = 512;
__global__ void __launch_bounds__(kXferThreads, 1) k_xfer(const __grid_constant__ XArgs A) {
  // dynamic smem: [staging buffers (if any op stages)] [word table]
  extern __shared__ __align__(128) uint8_t xsm[];
  __shared__ uint64_t mbar[kXferStageBufs];
  uint8_t* sbuf = xsm;
  int32_t* wt = reinterpret_cast<int32_t*>(xsm + A.wt_off);
  __shared__ uint64_t s_val;
  __shared__ int s_stop, s_gs;
  int op = 0;
  for (int i = 0; i < A.nops; i++)
    if ((int)blockIdx.x >= A.ops[i].cta0 && (int)blockIdx.x < A.ops[i].cta0 + A.ops[i].ncta) op = i;
  const XOp& X = A.ops[op];
  const int j = (int)blockIdx.x - X.cta0;
  if (X.kind == 2)
    for (int i = threadIdx.x; i < X.P.nwords; i += blockDim.x) wt[i] = X.P.wtab[i];
  if (X.kind == 4)
    for (int i = threadIdx.x; i < X.P.nwords; i += blockDim.x) wt[i] = X.P.wtab[i];
  if (X.kind == 6) {  // record-span maps after the per-warp buffers (same layout as cta_chunk)
    const RecGeo& R = X.rg;
    uint16_t* omap = reinterpret_cast<uint16_t*>(xsm + (blockDim.x >> 5) * (R.RB * R.spanB + R.RB * 8));
    if (X.role == 1) {
      switch (X.g) { case 4: rec_maps<true, 4>(R, omap); break; case 8: rec_maps<true, 8>(R, omap); break;
                     default: rec_maps<true, 16>(R, omap); break; }
    } else {
      switch (X.g) { case 4: rec_maps<false, 4>(R, omap); break; case 8: rec_maps<false, 8>(R, omap); break;
                     default: rec_maps<false, 16>(R, omap); break; }
    }
  }
  const int64_t C = X.chunk;
  const int D = X.depth;
  if (threadIdx.x == 0) s_stop = 0;
  __syncthreads();

  // Sub-rings: step k of the message covers stream bytes [kC, (k+1)C); sub-ring
  // js in [0, gs) carries [kC + js*Cs, kC + (js+1)*Cs), Cs = C/gs, through its own
  // D slots and flags, so every CTA pipelines on its own (no cross-CTA wait per
  // fragment).  The sender runs one CTA per sub-ring; receiver CTA j serves
  // sub-rings j, j+ncta, ...
  // Replicas: with an even depth, sub-ring js is served by `rep` CTAs that take alternate
  // fragments (fragment k -> replica k % rep; slot k % D belongs to one replica), so two
  // fragments of a sub-ring are in flight at once and each fragment's fixed cost (credit
  // poll, store completion, publication) overlaps the other's copy.
  int64_t n = X.n;
  int gs, rep;
  __shared__ int s_rep;
  if (X.role == 0) {
    rep = X.rep > 1 ? X.rep : 1;
    gs = X.ncta / rep;
    // ---- send role: header {seq, nbytes, gs, rep}, wait for "go" (receiver-driven, [L20:c3973])
    if (j == 0 && threadIdx.x == 0) {
      st_release_sys(X.hdr + 1, (uint64_t)n);
      st_release_sys(X.hdr + 2, (uint64_t)gs);
      st_release_sys(X.hdr + 3, (uint64_t)rep);
      st_release_sys(X.hdr, X.seq);
    }
    if (threadIdx.x == 0) {
      uint64_t v = 0;
      const uint64_t seq = X.seq;
      bool ok = spin(X.go, [seq](uint64_t x) { return (x & ~kAbort) >= seq; }, A.timeout_ns, X.err, &v);
      s_stop = !ok ? 2 : (v & kAbort) ? 1 : 0;
      if (s_stop == 1 && j == 0) atomicCAS(X.err, 0, XERR_TRUNCATE);
    }
    __syncthreads();
    if (s_stop == 2) return;
    if (s_stop == 1) n = 0;  // aborted: move nothing, carry the bases over
  } else {
    // ---- recv role: read the header, check capacity, send "go"
    if (threadIdx.x == 0) {
      uint64_t v = 0;
      const uint64_t seq = X.seq;
      bool ok = spin(X.hdr, [seq](uint64_t x) { return x >= seq; }, A.timeout_ns, X.err, &v);
      s_val = ok ? ld_acquire_sys(X.hdr + 1) : 0;
      s_gs = ok ? (int)ld_acquire_sys(X.hdr + 2) : 1;
      s_rep = ok ? (int)ld_acquire_sys(X.hdr + 3) : 1;
      s_stop = ok ? 0 : 2;
    }
    __syncthreads();
    if (s_stop == 2) return;
    n = (int64_t)s_val;
    gs = s_gs;
    rep = s_rep > 1 ? s_rep : 1;
    if (n > X.n) {
      if (j == 0 && threadIdx.x == 0) {
        atomicCAS(X.err, 0, XERR_TRUNCATE);
        st_release_sys(X.go, X.seq | kAbort);
      }
      n = 0;
    } else if (j == 0 && threadIdx.x == 0) {
      st_release_sys(X.go, X.seq);
    }
  }

  const int64_t Cs = C / gs;
  const int64_t K = (n + C - 1) / C;
  // this CTA's replica and sub-rings: sender CTA j = replica j / gs of sub-ring j % gs;
  // receiver CTAs split into rep groups of nsub (a receiver with fewer CTAs than
  // replicas serves every fragment)
  int myrep = 0, js0 = j, jstep = X.ncta;
  bool all_k = rep == 1;
  if (X.role == 0) {
    myrep = j / gs;
    js0 = j % gs;
    jstep = gs;
  } else if (X.ncta >= rep && rep > 1) {
    const int nsub = X.ncta / rep;
    myrep = j / nsub;
    js0 = j % nsub;
    jstep = nsub;
    if (myrep >= rep) js0 = gs;  // surplus CTA: no sub-ring
  } else {
    all_k = true;
  }
  for (int64_t k = 0; k < K; k++) {
    if (!all_k && (int)(k % rep) != myrep) continue;
    const int slot = (int)(k % D);
    const int64_t round = k / D;
    for (int js = js0; js < gs; js += jstep) {
      const int64_t off = k * C + (int64_t)js * Cs;
      if (off >= n) continue;
      const int64_t len = min(Cs, n - off);
      const int fi = js * D + slot;  // flag / base index of (sub-ring, slot)
      uint8_t* sl = X.ring + (int64_t)fi * Cs - off;  // stream byte `off` lands at the slot start
      const uint64_t base = X.base_in[fi] + (uint64_t)round * (uint64_t)Cs;
      if (threadIdx.x == 0) {
        uint64_t v;
        bool ok;
        const bool sl_ok = !(A.flags & 2);
        if (X.role == 0)
          ok = spin(X.ack + fi, [base](uint64_t x) { return x >= base; }, A.timeout_ns, X.err, &v, sl_ok);
        else {
          const uint64_t need = base + (uint64_t)len;
          ok = spin(X.ready + fi, [need](uint64_t x) { return x >= need; }, A.timeout_ns, X.err, &v, sl_ok);
        }
        s_stop = ok ? 0 : 2;
      }
      __syncthreads();
      if (s_stop) return;
      if (X.role == 0) cta_chunk<false>(X, sl, off, len, wt, sbuf, mbar);
      else cta_chunk<true>(X, sl, off, len, wt, sbuf, mbar);
      __syncthreads();
      if (threadIdx.x == 0) {
        // Publication: the CTA's stores (generic, and TMA bulk stores that thread 0 issued
        // and waited for) precede this thread's system-scope release through the barrier
        // above; the release is cumulative, so the peer's acquire of the counter sees them
        // (the message-passing pattern NCCL's simple protocol uses: barrier, acq_rel fence
        // at system scope, flag store).  The proxy fence orders the async-proxy writes with
        // the generic release.  A full SC fence (bit 2 of DT_XFER_FLAGS) cost 20-25 % of
        // the loopback exchange rate at 1-4 MiB fragments and is not needed for this pattern.
        if (A.flags & 4) __threadfence_system();
        if (X.kind == 4 && X.role == 0) asm volatile("fence.proxy.async.global;" ::: "memory");  // TMA stores
        red_release_sys_add(X.role == 0 ? X.ready + fi : X.ack + fi, (uint64_t)len);
      }
    }
  }
  // cumulative per-(sub-ring, slot) bytes after this message (read by the next
  // message's kernel from the other parity); every sub-ring is carried over
  for (int js = j; js < kMaxSub; js += X.ncta) {
    for (int s = threadIdx.x; s < D; s += blockDim.x) {
      uint64_t add = 0;
      if (js < gs)
        for (int64_t k = s; k < K; k += D) {
          const int64_t off = k * C + (int64_t)js * Cs;
          if (off < n) add += (uint64_t)min(Cs, n - off);
        }
      X.base_out[js * D + s] = X.base_in[js * D + s] + add;
    }
  }
}

// ------------------------------------------------------------------ NCCL (dlopen)
typedef struct { char internal[128]; } ncclUniqueId_t;
typedef void* ncclComm_t;
struct Nccl {
  void* h = nullptr;
  int (*GetUniqueId)(ncclUniqueId_t*) = nullptr;
  int (*CommInitRank)(ncclComm_t*, int, ncclUniqueId_t, int) = nullptr;
  int (*Send)(const void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  int (*Recv)(void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  int (*GroupStart)() = nullptr;
  int (*GroupEnd)() = nullptr;
  int (*CommDestroy)(ncclComm_t) = nullptr;
  const char* (*GetErrorString)(int) = nullptr;
};
static Nccl g_nccl;
static std::mutex g_nccl_mu;

static bool load_nccl() {
  std::lock_guard<std::mutex> g(g_nccl_mu);
  if (g_nccl.h) return true;
  const char* names[] = {"libnccl.so.2", "libnccl.so", nullptr};
  void* h = nullptr;
  // prefer the copy torch already loaded (same SONAME), else the pip wheel's, else the system one
  for (int i = 0; names[i] && !h; i++) h = dlopen(names[i], RTLD_NOW | RTLD_NOLOAD);
  if (!h && getenv("DT_NCCL_LIB")) h = dlopen(getenv("DT_NCCL_LIB"), RTLD_NOW);
  for (int i = 0; names[i] && !h; i++) h = dlopen(names[i], RTLD_NOW);
  if (!h) return false;
#define SYM(f, n) g_nccl.f = (decltype(g_nccl.f))dlsym(h, n)
  SYM(GetUniqueId, "ncclGetUniqueId");
  SYM(CommInitRank, "ncclCommInitRank");
  SYM(Send, "ncclSend");
  SYM(Recv, "ncclRecv");
  SYM(GroupStart, "ncclGroupStart");
  SYM(GroupEnd, "ncclGroupEnd");
  SYM(CommDestroy, "ncclCommDestroy");
  SYM(GetErrorString, "ncclGetErrorString");
#undef SYM
  if (!g_nccl.GetUniqueId || !g_nccl.CommInitRank || !g_nccl.Send || !g_nccl.Recv || !g_nccl.GroupStart ||
      !g_nccl.GroupEnd || !g_nccl.CommDestroy)
    return false;
  g_nccl.h = h;
  return true;
}

}  // namespace dt

using namespace dt;

// ------------------------------------------------------------------ comm object
struct HandleBlob {
  uint32_t magic;
  int32_t rank;
  int64_t pid;
  int32_t device;
  int32_t pad;
  uint64_t ring_ptr, flags_ptr;
  cudaIpcMemHandle_t ring_h, flags_h;
};
static const uint32_t kMagic = 0xD7A7C0DEu;

struct PendingOp {
  const void* sbuf;
  int64_t scount;
  dt_t stype;
  int dest;
  void* rbuf;
  int64_t rcount;
  dt_t rtype;
  int source;
};

struct dt_comm_s {
  int rank = 0, nranks = 1, device = 0;
  dt_xfer_opts o{};
  int nch = kMaxCh;
  uint8_t* ring = nullptr;
  uint64_t* flags = nullptr;
  uint64_t* bases = nullptr;  // [2 parities][2 dirs][nranks][nch][depth]
  size_t ring_bytes = 0, flag_words = 0;
  std::vector<uint8_t*> peer_ring;
  std::vector<uint64_t*> peer_flags;
  std::vector<bool> opened;
  bool connected = false;
  std::vector<uint64_t> send_seq, recv_seq;  // [nranks*nch]
  // group
  bool in_group = false;
  std::vector<PendingOp> pending;
  // NCCL mode
  ncclComm_t nccl = nullptr;
  cudaStream_t s_pack = nullptr, s_net = nullptr, s_unpack = nullptr;
  std::vector<cudaEvent_t> ev;
  uint8_t* stage = nullptr;  // send staging [kMaxOps][depth][chunk]
  uint8_t* rstage = nullptr; // recv staging
  int64_t* szbuf = nullptr;  // device size handshake buffers [2][kMaxOps]
  int64_t* szhost = nullptr; // pinned
  // layout helpers (uint64 flag words): per (peer, channel) kMaxSub*depth ready
  // counters, a 4-word header {seq, nbytes, sub-rings, replicas}, kMaxSub*depth ack
  // counters and a go word; then one error word.  The ring of a (source,
  // channel) pair is depth*chunk bytes, split among the sender's sub-rings.
  size_t per() const { return (size_t)kMaxSub * o.depth; }
  size_t pairs() const { return (size_t)nranks * nch; }
  size_t ready_idx(int src, int ch) const { return ((size_t)src * nch + ch) * per(); }
  size_t hdr_idx(int src, int ch) const { return pairs() * per() + ((size_t)src * nch + ch) * 4; }
  size_t ack_idx(int dst, int ch) const { return pairs() * (per() + 4) + ((size_t)dst * nch + ch) * per(); }
  size_t go_idx(int dst, int ch) const { return pairs() * (2 * per() + 4) + (size_t)dst * nch + ch; }
  size_t err_idx() const { return pairs() * (2 * per() + 5); }
  size_t ring_off(int src, int ch) const { return (((size_t)src * nch + ch) * o.depth) * (size_t)o.chunk_bytes; }
  uint64_t* base(int parity, int dir, int peer, int ch) const {
    return bases + ((((size_t)parity * 2 + dir) * nranks + peer) * nch + ch) * per();
  }
};

void dt::comm_info(dt_comm_t c, int* rank, int* nranks, int* device) {
  *rank = c->rank;
  *nranks = c->nranks;
  *device = c->device;
}

static dt_status cufail(cudaError_t e, const char* what) {
  set_error("%s: %s", what, cudaGetErrorString(e));
  return DT_ERR_CUDA;
}
#define CU(call)                                      \
  do {                                                \
    cudaError_t _e = (call);                          \
    if (_e != cudaSuccess) return cufail(_e, #call);  \
  } while (0)
#define NC(call)                                                                         \
  do {                                                                                   \
    int _r = (call);                                                                     \
    if (_r != 0) {                                                                       \
      set_error("%s: nccl error %d (%s)", #call, _r,                                     \
                g_nccl.GetErrorString ? g_nccl.GetErrorString(_r) : "?");                \
      return DT_ERR_NCCL;                                                                \
    }                                                                                    \
  } while (0)

static void fill_opts(dt_xfer_opts& o, const dt_xfer_opts* in) {
  o.chunk_bytes = 1 << 20;
  o.depth = 8;
  o.mode = DT_XFER_P2P;
  o.ctas = 0;
  o.flags = in ? in->flags : 0;
  if (in) {
    if (in->chunk_bytes > 0) o.chunk_bytes = in->chunk_bytes;
    if (in->depth > 0) o.depth = in->depth;
    o.mode = in->mode;
    o.ctas = in->ctas;
  }
  o.chunk_bytes = (o.chunk_bytes + 511) & ~int64_t(511);
}

extern "C" {

dt_status dt_nccl_unique_id(void* out128) {
  if (!out128) {
    set_error("dt_nccl_unique_id: NULL");
    return DT_ERR_ARG;
  }
  if (!load_nccl()) {
    set_error("NCCL library not found");
    return DT_ERR_NCCL;
  }
  ncclUniqueId_t id;
  NC(g_nccl.GetUniqueId(&id));
  std::memcpy(out128, &id, 128);
  return DT_OK;
}

dt_status dt_comm_init(int rank, int nranks, const void* nccl_unique_id, int device, const dt_xfer_opts* o,
                       dt_comm_t* out) {
  if (!out || nranks < 1 || rank < 0 || rank >= nranks || device < 0) {
    set_error("dt_comm_init: bad argument");
    return DT_ERR_ARG;
  }
  auto* c = new dt_comm_s;
  c->rank = rank;
  c->nranks = nranks;
  c->device = device;
  fill_opts(c->o, o);
  if (c->o.mode != DT_XFER_P2P && c->o.mode != DT_XFER_NCCL) {
    delete c;
    set_error("dt_comm_init: unknown mode");
    return DT_ERR_ARG;
  }
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) {
    delete c;
    return cufail(e, "cudaSetDevice");
  }
  c->ring_bytes = (size_t)nranks * c->nch * c->o.depth * (size_t)c->o.chunk_bytes;
  c->flag_words = c->err_idx() + 1;
  if (c->o.mode == DT_XFER_P2P) {
    e = cudaMalloc(&c->ring, c->ring_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&c->flags, c->flag_words * 8);
    if (e == cudaSuccess) e = cudaMemset(c->flags, 0, c->flag_words * 8);
    const size_t nb = (size_t)2 * 2 * c->pairs() * c->per();
    if (e == cudaSuccess) e = cudaMalloc(&c->bases, nb * 8);
    if (e == cudaSuccess) e = cudaMemset(c->bases, 0, nb * 8);
    if (e != cudaSuccess) {
      cudaFree(c->ring);
      cudaFree(c->flags);
      cudaFree(c->bases);
      delete c;
      return cufail(e, "dt_comm_init alloc");
    }
  } else {
    if (!load_nccl()) {
      delete c;
      set_error("dt_comm_init: NCCL library not found");
      return DT_ERR_NCCL;
    }
    if (!nccl_unique_id) {
      delete c;
      set_error("dt_comm_init: NCCL mode needs a unique id");
      return DT_ERR_ARG;
    }
    ncclUniqueId_t id;
    std::memcpy(&id, nccl_unique_id, 128);
    int r = g_nccl.CommInitRank(&c->nccl, nranks, id, rank);
    if (r != 0) {
      delete c;
      set_error("ncclCommInitRank failed: %d", r);
      return DT_ERR_NCCL;
    }
    const size_t st = (size_t)kMaxOps * c->o.depth * (size_t)c->o.chunk_bytes;
    e = cudaMalloc(&c->stage, st);
    if (e == cudaSuccess) e = cudaMalloc(&c->rstage, st);
    if (e == cudaSuccess) e = cudaMalloc(&c->szbuf, sizeof(int64_t) * 2 * kMaxOps);
    if (e == cudaSuccess) e = cudaMallocHost(&c->szhost, sizeof(int64_t) * 2 * kMaxOps);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s_pack, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s_net, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s_unpack, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
      delete c;
      return cufail(e, "dt_comm_init nccl alloc");
    }
    c->ev.resize((size_t)kMaxOps * c->o.depth * 3 + 2);
    for (auto& x : c->ev) cudaEventCreateWithFlags(&x, cudaEventDisableTiming);
  }
  c->peer_ring.assign(nranks, nullptr);
  c->peer_flags.assign(nranks, nullptr);
  c->opened.assign(nranks, false);
  c->send_seq.assign((size_t)nranks * c->nch, 0);
  c->recv_seq.assign((size_t)nranks * c->nch, 0);
  c->peer_ring[rank] = c->ring;
  c->peer_flags[rank] = c->flags;
  if (nranks == 1 || c->o.mode == DT_XFER_NCCL) c->connected = true;
  *out = c;
  return DT_OK;
}

dt_status dt_comm_local_handle(dt_comm_t c, void* out, size_t* nbytes) {
  if (!c || !nbytes) {
    set_error("dt_comm_local_handle: NULL");
    return DT_ERR_ARG;
  }
  if (!out || *nbytes < sizeof(HandleBlob)) {
    *nbytes = sizeof(HandleBlob);
    if (!out) return DT_OK;
    set_error("dt_comm_local_handle: buffer too small");
    return DT_ERR_ARG;
  }
  HandleBlob b;
  std::memset(&b, 0, sizeof(b));
  b.magic = kMagic;
  b.rank = c->rank;
  b.pid = (int64_t)getpid();
  b.device = c->device;
  b.ring_ptr = (uint64_t)(uintptr_t)c->ring;
  b.flags_ptr = (uint64_t)(uintptr_t)c->flags;
  if (c->o.mode == DT_XFER_P2P) {
    CU(cudaIpcGetMemHandle(&b.ring_h, c->ring));
    CU(cudaIpcGetMemHandle(&b.flags_h, c->flags));
  }
  std::memcpy(out, &b, sizeof(b));
  *nbytes = sizeof(b);
  return DT_OK;
}

dt_status dt_comm_connect(dt_comm_t c, const void* all, size_t per) {
  if (!c || !all || per < sizeof(HandleBlob)) {
    set_error("dt_comm_connect: bad argument");
    return DT_ERR_ARG;
  }
  if (c->o.mode != DT_XFER_P2P) {
    c->connected = true;
    return DT_OK;
  }
  CU(cudaSetDevice(c->device));
  const int64_t mypid = (int64_t)getpid();
  for (int r = 0; r < c->nranks; r++) {
    HandleBlob b;
    std::memcpy(&b, (const uint8_t*)all + (size_t)r * per, sizeof(b));
    if (b.magic != kMagic || b.rank != r) {
      set_error("dt_comm_connect: malformed handle of rank %d", r);
      return DT_ERR_ARG;
    }
    if (r == c->rank) continue;
    if (b.pid == mypid) {  // same process (e.g. several devices driven by one process)
      c->peer_ring[r] = (uint8_t*)(uintptr_t)b.ring_ptr;
      c->peer_flags[r] = (uint64_t*)(uintptr_t)b.flags_ptr;
      if (b.device != c->device) {
        cudaError_t e = cudaDeviceEnablePeerAccess(b.device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cufail(e, "cudaDeviceEnablePeerAccess");
        cudaGetLastError();
      }
      continue;
    }
    void *pr = nullptr, *pf = nullptr;
    CU(cudaIpcOpenMemHandle(&pr, b.ring_h, cudaIpcMemLazyEnablePeerAccess));
    CU(cudaIpcOpenMemHandle(&pf, b.flags_h, cudaIpcMemLazyEnablePeerAccess));
    c->peer_ring[r] = (uint8_t*)pr;
    c->peer_flags[r] = (uint64_t*)pf;
    c->opened[r] = true;
  }
  c->connected = true;
  return DT_OK;
}

dt_status dt_group_start(dt_comm_t c) {
  if (!c) {
    set_error("dt_group_start: NULL");
    return DT_ERR_ARG;
  }
  c->in_group = true;
  c->pending.clear();
  return DT_OK;
}

}  // extern "C"

// ------------------------------------------------------------------ issue
static int64_t lowp2u(uint64_t x) {
  if (x == 0) return 16;
  int64_t g = (int64_t)(x & (~x + 1));
  return g > 16 ? 16 : g;
}

// Fill the pack/unpack params of one side of an op (no chunk-specific fields).
static dt_status side_params(dt_t t, int64_t count, const void* nc, int64_t nbytes, int64_t chunk, XOp& X) {
  DeviceDesc* dd = nullptr;
  dt_status st = ensure_committed_on_device(t, &dd);
  if (st != DT_OK) return st;
  const Form& f = get_form(t);
  KLevels L;
  build_levels(f, dd, t, count, L);
  KP& P = X.P;
  std::memset(&P, 0, sizeof(P));
  P.nc = (const uint8_t*)nc;
  P.tsize = f.tsize();
  P.nblocks = (int64_t)f.bl.size();
  P.bd = dd->bd;
  P.bl = dd->bl;
  P.boff = dd->boff;
  P.bd0 = f.bd.empty() ? 0 : f.bd[0];
  P.bl0 = f.bl.empty() ? 0 : f.bl[0];
  P.nlev = L.n;
  for (int i = 0; i < L.n; i++) {
    P.cnt[i] = L.cnt[i];
    P.stride[i] = L.stride[i];
    P.table[i] = L.table[i];
    P.fcnt[i] = make_fd((uint64_t)L.cnt[i]);
  }
  P.ftsize = make_fd((uint64_t)P.tsize);
  int64_t g = 1;
  // chunk starts are multiples of `chunk` (a multiple of 512) and ring slots are aligned
  int kind = plan_kernel(f, L, (uint64_t)(uintptr_t)nc, 0, 0, nbytes, &g);
  if (kind == 6) {  // record spans: fragments start on 512-byte stream boundaries (16-byte aligned)
    if (!rec_geometry(f, L, (uint64_t)(uintptr_t)nc, 0, 0, nbytes, g, &X.rg) || getenv("DT_XFER_NOREC"))
      kind = g >= 8 ? 4 : 2;
  }
  if ((kind == 2 || kind == 4 || kind == 6 || kind == 7) && lowp2u((uint64_t)chunk) < g) kind = 1;
  if (kind == 4 && g < 8) kind = 2;
  if (kind == 7 && getenv("DT_XFER_NOSPAN")) kind = 1;
  // the block-window kernel (3) is not used inside the pipeline
  X.kind = (kind == 2 || kind == 4 || kind == 6 || kind == 7) ? kind : 1;
  if (X.kind == 7) P.fnb = make_fd((uint64_t)P.nblocks);
  X.single = P.nblocks == 1;
  X.g = (int32_t)g;
  if (X.kind == 2 || X.kind == 4) {
    const int32_t* wt = nullptr;
    st = ensure_wtab_pub(f, *dd, g, &wt);
    if (st != DT_OK) return st;
    P.wtab = wt;
    P.nwords = (int32_t)(f.tsize() / g);
  }
  return DT_OK;
}

// shared memory of a record-span op in the transfer kernel: per-warp record buffers and
// displacements, then the per-CTA map (layout as in cta_chunk / k_xfer)
static size_t rec_smem_bytes(const RecGeo& R, int g) {
  const size_t nwc = kXferThreads / 32;
  const size_t tab = std::max<size_t>((size_t)R.RB * R.nwr * 2, (size_t)(R.spanB / g) * 2);
  return nwc * ((size_t)R.RB * R.spanB + (size_t)R.RB * 8) + tab;
}

// CTAs per direction (capped by co-residency across the group's ops); 64 measured best for
// the loopback C3 exchange (738 vs 428 GB/s at 32, 16 MiB fragments)
static int default_ctas(const dt_comm_s* c) { return c->o.ctas > 0 ? c->o.ctas : 64; }

static dt_status issue_p2p(dt_comm_s* c, const std::vector<PendingOp>& ops, cudaStream_t s) {
  XArgs A;
  std::memset(&A, 0, sizeof(A));
  const char* to = getenv("DT_TIMEOUT_MS");
  A.timeout_ns = (int64_t)(to ? atoll(to) : 30000) * 1000000ll;
  A.flags = getenv("DT_XFER_FLAGS") ? atoi(getenv("DT_XFER_FLAGS")) : 0;
  int nops = 0, cta = 0;
  size_t smem = 0, rec_smem = 0;
  bool any_stage = false;
  std::vector<int> sch(c->nranks, 0), rch(c->nranks, 0);
  const int G = default_ctas(c);
  for (const auto& p : ops) {
    if (p.dest >= 0) {
      if (nops >= kMaxOps) { set_error("dt_sendrecv: too many ops in one group"); return DT_ERR_UNSUPPORTED; }
      const int ch = sch[p.dest]++;
      if (ch >= c->nch) { set_error("dt_sendrecv: more than %d messages to one peer in a group", c->nch); return DT_ERR_UNSUPPORTED; }
      XOp& X = A.ops[nops++];
      const int64_t n = p.scount * p.stype->size;
      dt_status st = side_params(p.stype, p.scount, p.sbuf, n, c->o.chunk_bytes, X);
      if (st != DT_OK) return st;
      X.role = 0;
      X.n = n;
      X.chunk = c->o.chunk_bytes;
      X.depth = c->o.depth;
      uint64_t* pf = c->peer_flags[p.dest];
      X.ring = c->peer_ring[p.dest] + c->ring_off(c->rank, ch);
      X.ready = pf + c->ready_idx(c->rank, ch);
      X.hdr = pf + c->hdr_idx(c->rank, ch);
      X.ack = c->flags + c->ack_idx(p.dest, ch);
      X.go = c->flags + c->go_idx(p.dest, ch);
      uint64_t& sq = c->send_seq[(size_t)p.dest * c->nch + ch];
      const int par = (int)(sq & 1);
      X.base_in = c->base(par, 0, p.dest, ch);
      X.base_out = c->base(par ^ 1, 0, p.dest, ch);
      X.seq = ++sq;
      X.err = reinterpret_cast<int32_t*>(c->flags + c->err_idx());
      if (X.kind == 2 || X.kind == 4) smem = std::max(smem, sizeof(int32_t) * (size_t)X.P.nwords);
      any_stage = any_stage || X.kind == 4;
      if (X.kind == 6) rec_smem = std::max(rec_smem, rec_smem_bytes(X.rg, X.g));
      if (X.kind == 7) rec_smem = std::max(rec_smem, (size_t)(kXferThreads / 32) * kSpanWarpSmem);
    }
    if (p.source >= 0) {
      if (nops >= kMaxOps) { set_error("dt_sendrecv: too many ops in one group"); return DT_ERR_UNSUPPORTED; }
      const int ch = rch[p.source]++;
      if (ch >= c->nch) { set_error("dt_sendrecv: more than %d messages from one peer in a group", c->nch); return DT_ERR_UNSUPPORTED; }
      XOp& X = A.ops[nops++];
      const int64_t cap = p.rcount * p.rtype->size;
      dt_status st = side_params(p.rtype, p.rcount, p.rbuf, cap, c->o.chunk_bytes, X);
      if (st != DT_OK) return st;
      X.role = 1;
      X.n = cap;
      X.chunk = c->o.chunk_bytes;
      X.depth = c->o.depth;
      uint64_t* pf = c->peer_flags[p.source];
      X.ring = c->ring + c->ring_off(p.source, ch);
      X.ready = c->flags + c->ready_idx(p.source, ch);
      X.hdr = c->flags + c->hdr_idx(p.source, ch);
      X.ack = pf + c->ack_idx(c->rank, ch);
      X.go = pf + c->go_idx(c->rank, ch);
      uint64_t& sq = c->recv_seq[(size_t)p.source * c->nch + ch];
      const int par = (int)(sq & 1);
      X.base_in = c->base(par, 1, p.source, ch);
      X.base_out = c->base(par ^ 1, 1, p.source, ch);
      X.seq = ++sq;
      X.err = reinterpret_cast<int32_t*>(c->flags + c->err_idx());
      if (X.kind == 2 || X.kind == 4) smem = std::max(smem, sizeof(int32_t) * (size_t)X.P.nwords);
      any_stage = any_stage || X.kind == 4;
      if (X.kind == 6) rec_smem = std::max(rec_smem, rec_smem_bytes(X.rg, X.g));
      if (X.kind == 7) rec_smem = std::max(rec_smem, (size_t)(kXferThreads / 32) * kSpanWarpSmem);
    }
  }
  if (nops == 0) return DT_OK;
  A.nops = nops;
  A.wt_off = (int32_t)std::max<size_t>(any_stage ? (size_t)kXferStageBufs * kStageTile : 0, (rec_smem + 127) & ~size_t(127));
  smem += (size_t)A.wt_off;
  if (smem > 48 * 1024) CU(cudaFuncSetAttribute(k_xfer, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  // every CTA must be co-resident: fit the per-op CTA count to the occupancy
  int occ = 0;
  CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_xfer, kXferThreads, smem));
  int sms = 0, dev = 0;
  CU(cudaGetDevice(&dev));
  CU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  const int per_op = std::max(1, std::min(G, occ * sms / nops));
  for (int i = 0; i < nops; i++) {
    int n_i = per_op;
    if (A.ops[i].role == 0) {  // rep CTAs per sub-ring; a sub-ring slot is C/gs bytes, a multiple of 512
      const int64_t C = A.ops[i].chunk;
      // replicas: each slot must belong to one replica, and each replica keeps >= 2 slots
      // (with one slot a replica waits a full round trip per fragment: C3 4 MiB, depth 2:
      // 441 -> 306 GB/s; depth 4 with 2 replicas: 436 -> 487, 1 MiB: 192 -> 296)
      // default: the most replicas (<= 4) that still leave each >= 2 slots (depth 8: 4
      // replicas, C3 1 MiB 415 GB/s; depth 4: 2 replicas, 300 GB/s)
      const char* rp = getenv("DT_XFER_REP");
      const int dep = A.ops[i].depth;
      int rep = rp ? std::max(1, atoi(rp)) : 4;
      if (!rp) {
        const int64_t K = (A.ops[i].n + C - 1) / C;  // fragments: replicas beyond K would idle
        while (rep > 1 && (dep % rep != 0 || dep / rep < 2 || rep > K)) rep /= 2;
      }
      if (dep % rep != 0 || dep / rep < 2 || per_op < rep) rep = 1;
      int g = 1;
      while (g * 2 * rep <= per_op && g * 2 <= kMaxSub && C % ((int64_t)g * 2 * 512) == 0) g *= 2;
      n_i = g * rep;
      A.ops[i].rep = rep;
    }
    A.ops[i].cta0 = cta;
    A.ops[i].ncta = n_i;
    cta += n_i;
  }
  // every CTA of both roles must be co-resident (they wait on each other): cooperative launch
  void* args[] = {&A};
  CU(cudaLaunchCooperativeKernel((void*)k_xfer, dim3(cta), dim3(kXferThreads), args, smem, s));
  return DT_OK;
}

// NCCL mode: size handshake, then per chunk round: pack -> send/recv -> unpack,
// double-buffered over `depth` staging slots on three internal streams.
static dt_status issue_nccl(dt_comm_s* c, const std::vector<PendingOp>& ops, cudaStream_t s) {
  const int64_t C = c->o.chunk_bytes;
  const int D = c->o.depth;
  std::vector<const PendingOp*> sends, recvs;
  for (const auto& p : ops) {
    if (p.dest >= 0) sends.push_back(&p);
    if (p.source >= 0) recvs.push_back(&p);
  }
  if ((int)sends.size() > kMaxOps || (int)recvs.size() > kMaxOps) {
    set_error("dt_sendrecv: too many ops in one group");
    return DT_ERR_UNSUPPORTED;
  }
  // handshake: exchange byte counts (the receiver learns n, checks capacity)
  for (size_t i = 0; i < sends.size(); i++) c->szhost[i] = sends[i]->scount * sends[i]->stype->size;
  CU(cudaMemcpyAsync(c->szbuf, c->szhost, sizeof(int64_t) * sends.size(), cudaMemcpyHostToDevice, s));
  NC(g_nccl.GroupStart());
  for (size_t i = 0; i < sends.size(); i++) NC(g_nccl.Send(c->szbuf + i, 8, 1 /*uint8*/, sends[i]->dest, c->nccl, s));
  for (size_t i = 0; i < recvs.size(); i++)
    NC(g_nccl.Recv(c->szbuf + kMaxOps + i, 8, 1, recvs[i]->source, c->nccl, s));
  NC(g_nccl.GroupEnd());
  CU(cudaMemcpyAsync(c->szhost + kMaxOps, c->szbuf + kMaxOps, sizeof(int64_t) * recvs.size(),
                     cudaMemcpyDeviceToHost, s));
  CU(cudaStreamSynchronize(s));
  std::vector<int64_t> sn(sends.size()), rn(recvs.size());
  for (size_t i = 0; i < sends.size(); i++) sn[i] = c->szhost[i];
  for (size_t i = 0; i < recvs.size(); i++) {
    rn[i] = c->szhost[kMaxOps + i];
    if (rn[i] > recvs[i]->rcount * recvs[i]->rtype->size) {
      set_error("dt_sendrecv: message of %lld bytes truncated by a %lld-byte receive", (long long)rn[i],
                (long long)(recvs[i]->rcount * recvs[i]->rtype->size));
      return DT_ERR_TRUNCATE;
    }
  }
  int64_t K = 0;
  for (auto x : sn) K = std::max(K, (x + C - 1) / C);
  for (auto x : rn) K = std::max(K, (x + C - 1) / C);
  cudaEvent_t* ev = c->ev.data();
  auto ev_packed = [&](int slot) { return ev[slot]; };
  auto ev_net = [&](int slot) { return ev[D + slot]; };
  auto ev_unpacked = [&](int slot) { return ev[2 * D + slot]; };
  cudaEvent_t ev_start = ev[3 * D], ev_end = ev[3 * D + 1];
  CU(cudaEventRecord(ev_start, s));
  CU(cudaStreamWaitEvent(c->s_pack, ev_start, 0));
  CU(cudaStreamWaitEvent(c->s_net, ev_start, 0));
  CU(cudaStreamWaitEvent(c->s_unpack, ev_start, 0));
  const size_t slot_span = (size_t)kMaxOps * C;
  for (int64_t k = 0; k < K; k++) {
    const int slot = (int)(k % D);
    if (k >= D) CU(cudaStreamWaitEvent(c->s_pack, ev_net(slot), 0));  // staging slot sent
    for (size_t i = 0; i < sends.size(); i++) {
      int64_t pos = k * C, len = std::min<int64_t>(C, sn[i] - pos);
      if (len <= 0) continue;
      dt_status st = dt_pack(sends[i]->stype, sends[i]->scount, sends[i]->sbuf, c->stage + slot * slot_span + i * C,
                             pos, &len, c->s_pack);
      if (st != DT_OK) return st;
    }
    CU(cudaEventRecord(ev_packed(slot), c->s_pack));
    CU(cudaStreamWaitEvent(c->s_net, ev_packed(slot), 0));
    if (k >= D) CU(cudaStreamWaitEvent(c->s_net, ev_unpacked(slot), 0));  // receive slot free
    NC(g_nccl.GroupStart());
    for (size_t i = 0; i < sends.size(); i++) {
      int64_t len = std::min<int64_t>(C, sn[i] - k * C);
      if (len > 0) NC(g_nccl.Send(c->stage + slot * slot_span + i * C, (size_t)len, 1, sends[i]->dest, c->nccl, c->s_net));
    }
    for (size_t i = 0; i < recvs.size(); i++) {
      int64_t len = std::min<int64_t>(C, rn[i] - k * C);
      if (len > 0)
        NC(g_nccl.Recv(c->rstage + slot * slot_span + i * C, (size_t)len, 1, recvs[i]->source, c->nccl, c->s_net));
    }
    NC(g_nccl.GroupEnd());
    CU(cudaEventRecord(ev_net(slot), c->s_net));
    CU(cudaStreamWaitEvent(c->s_unpack, ev_net(slot), 0));
    for (size_t i = 0; i < recvs.size(); i++) {
      int64_t pos = k * C, len = std::min<int64_t>(C, rn[i] - pos);
      if (len <= 0) continue;
      dt_status st = dt_unpack(recvs[i]->rtype, recvs[i]->rcount, c->rstage + slot * slot_span + i * C,
                               recvs[i]->rbuf, pos, &len, c->s_unpack);
      if (st != DT_OK) return st;
    }
    CU(cudaEventRecord(ev_unpacked(slot), c->s_unpack));
  }
  // join: the caller's stream waits for all three internal streams
  CU(cudaEventRecord(ev_end, c->s_pack));
  CU(cudaStreamWaitEvent(s, ev_end, 0));
  CU(cudaEventRecord(ev_end, c->s_net));
  CU(cudaStreamWaitEvent(s, ev_end, 0));
  CU(cudaEventRecord(ev_end, c->s_unpack));
  CU(cudaStreamWaitEvent(s, ev_end, 0));
  return DT_OK;
}

static dt_status validate(dt_comm_s* c, const PendingOp& p) {
  if (p.dest >= c->nranks || p.source >= c->nranks || p.dest < -1 || p.source < -1) {
    set_error("dt_sendrecv: rank out of range");
    return DT_ERR_ARG;
  }
  if (p.dest >= 0) {
    if (!p.stype || p.scount < 0 || (!p.sbuf && p.scount * p.stype->size > 0)) {
      set_error("dt_sendrecv: bad send arguments");
      return DT_ERR_ARG;
    }
    if (!p.stype->committed) {
      set_error("dt_sendrecv: send type not committed");
      return DT_ERR_NOT_COMMITTED;
    }
  }
  if (p.source >= 0) {
    if (!p.rtype || p.rcount < 0 || (!p.rbuf && p.rcount * p.rtype->size > 0)) {
      set_error("dt_sendrecv: bad receive arguments");
      return DT_ERR_ARG;
    }
    if (!p.rtype->committed) {
      set_error("dt_sendrecv: receive type not committed");
      return DT_ERR_NOT_COMMITTED;
    }
  }
  if (!c->connected) {
    set_error("dt_sendrecv: dt_comm_connect() not called");
    return DT_ERR_ARG;
  }
  return DT_OK;
}

// Loopback (dest = source = this rank, the paper's "1GPU" case [L26:c1686]) in
// P2P mode goes through the fused datatype -> datatype copy (f1): no ring, no
// flags, each byte moves once.  The k-th send-to-self of a call/group matches the
// k-th receive-from-self.  opts.flags bit 0 keeps loopback on the ring pipeline.
static dt_status issue(dt_comm_s* c, const std::vector<PendingOp>& ops_in, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (c->o.mode == DT_XFER_NCCL) return issue_nccl(c, ops_in, s);
  if (c->o.flags & 1) return issue_p2p(c, ops_in, s);
  std::vector<PendingOp> ops = ops_in;
  std::vector<size_t> sends, recvs;
  for (size_t i = 0; i < ops.size(); i++) {
    if (ops[i].dest == c->rank) sends.push_back(i);
    if (ops[i].source == c->rank) recvs.push_back(i);
  }
  for (size_t k = 0; k < std::min(sends.size(), recvs.size()); k++) {
    PendingOp& a = ops[sends[k]];
    PendingOp& b = ops[recvs[k]];
    dt_status st = dt_copy(a.stype, a.scount, a.sbuf, b.rtype, b.rcount, b.rbuf, stream);
    if (st != DT_OK) return st;
    a.dest = -1;
    b.source = -1;
  }
  return issue_p2p(c, ops, s);
}

extern "C" {

dt_status dt_sendrecv(const void* sbuf, int64_t scount, dt_t stype, int dest, void* rbuf, int64_t rcount, dt_t rtype,
                      int source, dt_comm_t c, const dt_xfer_opts* o, void* stream) {
  if (!c) {
    set_error("dt_sendrecv: NULL comm");
    return DT_ERR_ARG;
  }
  if (o && ((o->chunk_bytes > 0 && ((o->chunk_bytes + 511) & ~int64_t(511)) != c->o.chunk_bytes) ||
            (o->depth > 0 && o->depth != c->o.depth) || o->mode != c->o.mode)) {
    set_error("dt_sendrecv: opts differ from the comm's (chunk/depth/mode are fixed at dt_comm_init)");
    return DT_ERR_UNSUPPORTED;
  }
  PendingOp p{sbuf, scount, stype, dest, rbuf, rcount, rtype, source};
  dt_status st = validate(c, p);
  if (st != DT_OK) return st;
  if (c->in_group) {
    c->pending.push_back(p);
    return DT_OK;
  }
  std::vector<PendingOp> one{p};
  return issue(c, one, stream);
}

dt_status dt_group_end(dt_comm_t c, void* stream) {
  if (!c || !c->in_group) {
    set_error("dt_group_end: no open group");
    return DT_ERR_ARG;
  }
  c->in_group = false;
  std::vector<PendingOp> ops;
  ops.swap(c->pending);
  return issue(c, ops, stream);
}

dt_status dt_comm_check(dt_comm_t c) {
  if (!c) {
    set_error("dt_comm_check: NULL");
    return DT_ERR_ARG;
  }
  if (!c->flags) return DT_OK;
  int32_t e = 0;
  CU(cudaMemcpy(&e, c->flags + c->err_idx(), sizeof(e), cudaMemcpyDeviceToHost));
  if (e == 0) return DT_OK;
  int32_t z = 0;
  CU(cudaMemcpy(c->flags + c->err_idx(), &z, sizeof(z), cudaMemcpyHostToDevice));
  if (e == XERR_TRUNCATE) {
    set_error("dt_sendrecv: receive capacity smaller than the message (truncation)");
    return DT_ERR_TRUNCATE;
  }
  set_error("dt_sendrecv: device-side wait for a peer flag timed out");
  return DT_ERR_TIMEOUT;
}

dt_status dt_comm_free(dt_comm_t* pc) {
  if (!pc || !*pc) {
    set_error("dt_comm_free: NULL");
    return DT_ERR_ARG;
  }
  dt_comm_s* c = *pc;
  cudaSetDevice(c->device);
  for (int r = 0; r < c->nranks; r++) {
    if (!c->opened[r]) continue;
    cudaIpcCloseMemHandle(c->peer_ring[r]);
    cudaIpcCloseMemHandle(c->peer_flags[r]);
  }
  cudaFree(c->ring);
  cudaFree(c->flags);
  cudaFree(c->bases);
  cudaFree(c->stage);
  cudaFree(c->rstage);
  cudaFree(c->szbuf);
  if (c->szhost) cudaFreeHost(c->szhost);
  for (auto e : c->ev) cudaEventDestroy(e);
  if (c->s_pack) cudaStreamDestroy(c->s_pack);
  if (c->s_net) cudaStreamDestroy(c->s_net);
  if (c->s_unpack) cudaStreamDestroy(c->s_unpack);
  if (c->nccl && g_nccl.CommDestroy) g_nccl.CommDestroy(c->nccl);
  delete c;
  *pc = nullptr;
  return DT_OK;
}

}  // extern "C"
