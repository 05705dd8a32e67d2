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
//    send-role CTAs pack pieces of fragment k straight into the receiver's ring
//    slot k%D in peer HBM over NVLink, then publish each piece with a system-scope
//    release store of a tag (seq, round) into the receiver's ready flag; the
//    receive-role CTAs spin (ld.acquire.sys) on their local ready flags, unpack the
//    piece into the user's layout and release the tag into the sender's ack flag.
//    Chunk != launch: the chunk size only sets flow-control granularity.  The
//    receiver posts {capacity, seq} ("start packing") at kernel start; the sender
//    answers with the header {seq, n | abort, pieces, teams}.  The grid is sized to
//    the message (pieces of >= 32 KiB, teams of CTAs taking alternate fragments).
//  * NCCL mode: double-buffered chunks: pack(k) -> ncclSend/ncclRecv -> unpack(k)
//    on three internal streams with per-slot events.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <unistd.h>

#include <algorithm>
#include <cstddef>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "dt_device.cuh"
#include "dt_internal.h"

namespace dt {

constexpr int kMaxOps = 16;
constexpr int kMaxCh = 6;    // concurrent messages per (pair, direction) inside one group
constexpr int kMaxSub = 64;  // pieces (sub-rings) per fragment
constexpr int kMaxDepth = 256;  // ring slots per (pair, channel)
// CTA layout: warp 0 = control warp; then kGroups copy groups of kGroupWarps warps.
// Piece i of a CTA goes to group i % 2, so two pieces are copied concurrently and a
// piece's fixed latencies (TMA completion, barriers) overlap the other's copy.
constexpr int kGroups = 2, kGroupWarps = 8;
constexpr int kCopyWarps = kGroups * kGroupWarps;
constexpr int kGroupThreads = kGroupWarps * 32;
constexpr int kXferThreads = 32 + kCopyWarps * 32;
constexpr uint64_t kAbort = 1ull << 63;

// Flag values are tags: (message sequence number << 32) | (round + 1).  They only
// grow on a (pair, channel), so a waiter compares with >= and nothing is ever reset
// or carried between messages.  Round r of slot s is fragment r*D + s.
__host__ __device__ __forceinline__ uint64_t xtag(uint64_t seq, int64_t round) {
  return (seq << 32) | (uint64_t)(round + 1);
}

struct XOp {
  KP P;            // pack (send role) or unpack (recv role) over the user's layout
  int32_t role;    // 0 send, 1 recv
  int32_t kind;    // 1 segment walk, 2 word table, 4 smem/TMA staging, 6 record spans, 7 block spans
  int32_t single;  // segment walk over a single-block template
  int32_t g;       // word granularity
  int64_t n;       // send: bytes; recv: capacity in bytes
  int64_t chunk;   // C: fragment bytes (one ring slot)
  int32_t depth, cta0, ncta;
  int32_t gs, rep;  // send role: pieces per fragment, teams (fragment k -> team k % rep)
  int32_t sys;      // flag scope: 1 = system (peer on another GPU), 0 = gpu (same device)
  uint8_t* ring;   // slot 0 of the (pair, channel) ring (send: peer memory; recv: local)
  uint64_t* ready; // [depth][kMaxSub] tags  send: peer; recv: local
  uint64_t* ack;   // [depth][kMaxSub] tags  send: local; recv: peer
  uint64_t* hdr;   // [4] {seq, nbytes, gs, rep}  send: peer; recv: local
  uint64_t* go;    // [2] {consumed seq, aborted seq}  send: local; recv: peer
  uint32_t* done;  // local counter of this op's CTAs finished with the message (the last one
                   // advances *seqp and, receiving, posts consumed)
  uint64_t* seqp;  // local: the channel's last message sequence number in this role (device-
                   // resident, so a captured CUDA graph replays with fresh numbers)
  int32_t* err;
  RecGeo rg;       // kind 6: record-span geometry (per-fragment element range set on the device)
};

// Kernel parameters: NOPS ops (a single dt_sendrecv has <= 2; a group up to kMaxOps).
// Each XOp is ~700 bytes, and the kernel parameters travel with every launch: the
// 2-op instantiation keeps a single exchange's launch small.
template <int NOPS>
struct XArgsT {
  int32_t nops;
  int32_t wt_off;  // byte offset of the word table in dynamic smem (after the staging buffers)
  int32_t flags;   // DT_XFER_FLAGS: 2 = no sleep in polls, 4 = SC system fence before each flag, 8 = no proxy
                   // fence before TMA reads of a slot, 16 = one piece outstanding, 64 = publish every ack
  int32_t pad2;
  int64_t timeout_ns;
  uint64_t* trace;  // diagnostics (DT_XFER_TRACE): per-piece globaltimer stamps of the first CTAs
  XOp ops[NOPS];
};
typedef XArgsT<kMaxOps> XArgs;
constexpr int kTraceCtas = 4, kTracePieces = 64, kTracePts = 6;
// points: 0 control starts waiting for the piece's flag, 1 flag acquired, 2 copy seen
// done, 3 flag released, 4 copy group starts the piece, 5 copy group done
template <int NOPS>
__device__ __forceinline__ void xtrace(const XArgsT<NOPS>& A, int op, int j, int idx, int point) {
  if (A.trace && j < kTraceCtas && idx < kTracePieces)
    *(volatile uint64_t*)&A.trace[(((size_t)op * kTraceCtas + j) * kTracePieces + idx) * kTracePts + point] = gtimer();
}

// ---- per-family piece copies.  Each is a separate (noinline) function so that
// ptxas compiles the families one at a time instead of one giant kernel body.
// The op's parameters stay in the grid-constant bank (X refers to it).
template <bool UNPACK, bool SINGLE>
__device__ __noinline__ void xc_seg(const XOp& X, uint8_t* cb, int64_t a, int64_t b, int lane) {
  constexpr int POL = UNPACK ? LD_CG : LD_CS;  // ring slots are rewritten by the peer: bypass L1
  seg_range<UNPACK, SINGLE, POL>(X.P, cb, a, b, lane);
}

template <bool UNPACK, int G>
__device__ __noinline__ void xc_rec(const XOp& X, uint8_t* cb, int64_t lo, int64_t hb, uint8_t* sbuf, int w,
                                    int nwc, int cw) {
  constexpr int POL = UNPACK ? LD_CG : LD_CS;
  const KP& P = X.P;
  RecGeo R = X.rg;
  R.e_lo = lo / P.tsize;
  R.e_hi = (hb + P.tsize - 1) / P.tsize;
  R.b0 = R.e_lo & ~int64_t(31);
  R.nbatch = (R.e_hi - R.b0 + R.RB - 1) / R.RB;
  // per-copy-warp buffers (cw: the warp's index among all copy warps, layout as set up in
  // k_xfer); the work is split over the nwc warps of the group (w: index in the group)
  const int lane = threadIdx.x & 31;
  uint8_t* buf = sbuf + cw * (R.RB * R.spanB);
  int64_t* sd = reinterpret_cast<int64_t*>(sbuf + kCopyWarps * (R.RB * R.spanB)) + cw * R.RB;
  uint16_t* omap = reinterpret_cast<uint16_t*>(sbuf + kCopyWarps * (R.RB * R.spanB) + kCopyWarps * R.RB * 8);
  rec_range<UNPACK, G, POL>(P, R, cb, lo, hb, buf, sd, omap, w, nwc, lane);
}

template <bool UNPACK, int G>
__device__ __noinline__ void xc_span(const XOp& X, uint8_t* cb, int64_t a, int64_t b, uint8_t* sm, int lane) {
  constexpr int POL = UNPACK ? LD_CG : LD_CS;
  const PlanEnt st = span_start(X.P, a, lane);
  span_range<UNPACK, G, POL>(X.P, cb, st, b, lane, sm);
}

template <bool UNPACK, int G>
__device__ __noinline__ void xc_stage(const XOp& X, uint8_t* cb, const int32_t* wt, int64_t lo, int64_t bh,
                                      uint8_t* sbuf, uint64_t* mbar, int ctid, int cnthr, int bar, int64_t tb) {
  if (UNPACK) stage_unpack<G, kXferStageBufs>(X.P, cb, wt, lo, bh, sbuf, mbar, ctid, cnthr, bar, tb);
  else if (X.sys) stage_pack<G, kXferStageBufs, true>(X.P, cb, wt, lo, bh, sbuf, ctid, cnthr, bar);  // peer GPU
  else stage_pack<G, kXferStageBufs>(X.P, cb, wt, lo, bh, sbuf, ctid, cnthr, bar);
}

template <bool UNPACK, int G>
__device__ __noinline__ void xc_word(const XOp& X, uint8_t* cb, int64_t lo, int64_t hi, const int32_t* wt, int ctid,
                                     int cnthr) {
  constexpr int POL = UNPACK ? LD_CG : LD_CS;
  // few CTAs carry the whole transfer: keep 4 vectors per thread in flight (480 threads: 30 KiB/CTA)
  word_range<UNPACK, G, 16, POL, (G >= 4 ? 4 : 2)>(X.P, cb, lo, hi, wt, ctid, cnthr);
}

// pack or unpack stream bytes [lo, lo+len) of one piece with copy group g (warps
// 1 + 8g .. 8 + 8g of the CTA; warp 0 is the control warp).  cb: the slot base such
// that stream byte x of the message lives at cb + x.  sbuf: the CTA's dynamic smem
// (per-warp buffers of kinds 6/7, or this group's staging tiles for kind 4); mbar:
// this group's TMA mbarriers.
template <bool UNPACK>
__device__ __forceinline__ void cta_piece(const XOp& X, uint8_t* cb, int64_t lo, int64_t len, const int32_t* wt,
                                          uint8_t* sbuf, uint64_t* mbar, int g, int64_t& tb) {
  const int64_t hi = lo + len;
  const int cw = (threadIdx.x >> 5) - 1;  // copy warp index among all copy warps
  const int nwc = kGroupWarps, w = cw - g * kGroupWarps, lane = threadIdx.x & 31;
  const int ctid = threadIdx.x - 32 - g * kGroupThreads, cnthr = kGroupThreads, bar = 1 + g;
  if (X.kind == 6) {  // record spans: the copy warps take RB-record batches of the piece
    const int64_t hb = hi - len % X.g;  // a ragged tail (< G bytes, last piece) is walked below
    if (lo < hb) {
      switch (X.g) {
        case 4: xc_rec<UNPACK, 4>(X, cb, lo, hb, sbuf, w, nwc, cw); break;
        case 8: xc_rec<UNPACK, 8>(X, cb, lo, hb, sbuf, w, nwc, cw); break;
        default: xc_rec<UNPACK, 16>(X, cb, lo, hb, sbuf, w, nwc, cw); break;
      }
    }
    if (hb < hi && w == nwc - 1) xc_seg<UNPACK, false>(X, cb, hb, hi, lane);
    return;
  }
  if (X.kind == 7) {  // block spans: the copy warps take equal 16-byte-multiple slices of the piece
    const int64_t body = len - len % X.g;
    int64_t per = (body + nwc - 1) / nwc;
    per = (per + 15) & ~int64_t(15);
    const int64_t a = lo + (int64_t)w * per, b = min(a + per, lo + body);
    if (a < b) {
      uint8_t* sm = sbuf + (size_t)cw * kSpanWarpSmem;
      switch (X.g) {
        case 4: xc_span<UNPACK, 4>(X, cb, a, b, sm, lane); break;
        case 8: xc_span<UNPACK, 8>(X, cb, a, b, sm, lane); break;
        default: xc_span<UNPACK, 16>(X, cb, a, b, sm, lane); break;
      }
    }
    if (body < len && w == nwc - 1) xc_seg<UNPACK, false>(X, cb, lo + body, hi, lane);
    return;
  }
  if (X.kind == 4) {  // smem/TMA staging: bulk store into the (peer) ring slot / bulk load from it
    const int64_t bh = hi - len % X.g;
    uint8_t* gbuf = sbuf + (size_t)g * kXferStageBufs * kStageTile;
    if (X.g == 4) xc_stage<UNPACK, 4>(X, cb, wt, lo, bh, gbuf, mbar, ctid, cnthr, bar, tb);
    else if (X.g == 8) xc_stage<UNPACK, 8>(X, cb, wt, lo, bh, gbuf, mbar, ctid, cnthr, bar, tb);
    else xc_stage<UNPACK, 16>(X, cb, wt, lo, bh, gbuf, mbar, ctid, cnthr, bar, tb);
    tb += (bh - lo + kStageTile - 1) / kStageTile;  // tiles through this group's mbarriers
    if (bh < hi) {
      group_sync(bar, cnthr);
      if (w == 0) xc_seg<UNPACK, false>(X, cb, bh, hi, lane);
    }
    // the TMA bulk stores (async proxy) of the piece precede the control warp's release
    if (!UNPACK && !X.sys && ctid == 0) asm volatile("fence.proxy.async.global;" ::: "memory");
    return;
  }
  if (X.kind == 2) {
    const int64_t body = len - len % X.g;
    switch (X.g) {
      case 1: xc_word<UNPACK, 1>(X, cb, lo, lo + body, wt, ctid, cnthr); break;
      case 2: xc_word<UNPACK, 2>(X, cb, lo, lo + body, wt, ctid, cnthr); break;
      case 4: xc_word<UNPACK, 4>(X, cb, lo, lo + body, wt, ctid, cnthr); break;
      case 8: xc_word<UNPACK, 8>(X, cb, lo, lo + body, wt, ctid, cnthr); break;
      default: xc_word<UNPACK, 16>(X, cb, lo, lo + body, wt, ctid, cnthr); break;
    }
    if (body < len && w == 0) xc_seg<UNPACK, false>(X, cb, lo + body, hi, lane);
    return;
  }
  int64_t per = (len + nwc - 1) / nwc;
  per = (per + 127) & ~int64_t(127);
  const int64_t a = lo + (int64_t)w * per, b = min(a + per, hi);
  if (a < b) {
    if (X.single) xc_seg<UNPACK, true>(X, cb, a, b, lane);
    else xc_seg<UNPACK, false>(X, cb, a, b, lane);
  }
}

// The pieces one CTA handles, in fragment order (32-bit index math, slot and round
// kept incrementally).  Send role: CTA j = (team j / gs, piece j % gs), fragments
// j/gs, j/gs + rep, ...  Receive role: pairs j, j + ncta, ... (one pair per CTA
// when ncta >= pairs).  The control warp and the copy warps walk the same sequence.
struct PieceIt {
  int64_t n, C, Cs;
  int K, D, gs, gu, rep, ncta, j, jstep, kstep, k, js, slot, round;
  bool one;
  // gs: pieces per ring slot (layout, Cs = C/gs); gu: pieces of a fragment in use
  // (fewer than gs when the whole message is shorter than one slot)
  __device__ __forceinline__ bool init(int role, int64_t n_, int64_t C_, int D_, int gs_, int rep_, int ncta_, int j_) {
    n = n_; C = C_; D = D_; gs = gs_; rep = rep_; ncta = ncta_; j = j_;
    // (one thread runs this on the critical path of a short message: 32-bit arithmetic
    // where the values allow -- gs is a power of two, min(n, C) <= C < 2^31)
    Cs = C >> (__ffs(gs) - 1);
    K = (int)((n + C - 1) / C);
    gu = (int)min((uint32_t)gs, ((uint32_t)(n < C ? n : C) + (uint32_t)Cs - 1u) / (uint32_t)Cs);
    if (gu < 1) gu = 1;
    const int npairs = gu * rep;
    one = ncta >= npairs;  // (either role: fewer CTAs than pairs take pairs j, j + ncta, ...)
    if (one && j >= npairs) return false;
    kstep = one ? rep : 1;
    jstep = one ? gu : ncta;
    k = one ? j / gu : 0;
    slot = k % D;
    round = k / D;
    js = first_js();
    return settle();
  }
  __device__ __forceinline__ int first_js() const {
    return one ? j % gu : (((j - (k % rep) * gu) % ncta) + ncta) % ncta;
  }
  // advance to a valid (k, js) at or after the current one; false at the end
  __device__ __forceinline__ bool settle() {
    while (k < K) {
      if (js < gu && (int64_t)k * C + (int64_t)js * Cs < n) return true;
      k += kstep;
      slot += kstep;
      while (slot >= D) { slot -= D; round++; }
      if (k < K) js = first_js();
    }
    return false;
  }
  __device__ __forceinline__ bool next() {
    js += jstep;
    return settle();
  }
  __device__ __forceinline__ int64_t off() const { return (int64_t)k * C + (int64_t)js * Cs; }
  __device__ __forceinline__ int64_t len() const { return min(Cs, n - off()); }
  __device__ __forceinline__ int fi() const { return slot * kMaxSub + js; }
};

// One persistent kernel per dt_sendrecv / dt_group: send-role and receive-role CTAs
// of every op (co-resident: cooperative launch).
//
// Message protocol on a (pair, channel), sequence number seq:
//  * the sender does not wait for the receiver's kernel: the receiver posted
//    "consumed = seq-1" when its previous kernel on the channel finished (the last
//    of its CTAs, [L20:c4133]), so every ring slot is free; sender CTA 0 writes the
//    header {seq, n, gs, rep} and the pieces start at once;
//  * the message is K = ceil(n/C) fragments ("unpack fragment i", [L20:c3380]);
//    fragment k uses ring slot k % D, is split into gs pieces of C/gs bytes (gu of
//    them used: fewer for a message shorter than C), and belongs to team k % rep.
//    Sender CTA (team t, piece js) packs its pieces of t's fragments straight into
//    the receiver's slot in peer HBM and publishes each with a release store of the
//    tag into ready[slot][js]; before reusing a slot (round r > 0) it waits for
//    ack[slot][js] >= tag(seq, r-1);
//  * receiver CTAs read the header, take (team, piece) pairs round-robin, wait for
//    ready with an acquire, unpack the piece from local HBM and release the tag into
//    the sender's ack[slot][js];
//  * truncation (n > the receive capacity, [L26:c4404], reading A12) is decided by
//    the receiver from the header before any byte reaches the receive buffer: it
//    reports DT_ERR_TRUNCATE (an MPI receive-side error), unpacks nothing and posts
//    "aborted = seq" so a sender waiting for a slot stops (the bytes it staged are
//    never read; the next message's tags supersede their flags).
// Flags are written by exactly one CTA, so plain release stores suffice, and since
// tags only grow nothing is carried between messages.
// A CTA finished its part of message seq (every piece it owns copied and its flags
// released, by this thread).  The last CTA of the op advances the channel's device-
// resident sequence number and, receiving, posts "consumed = seq" to the sender --
// the ring is free for the next message on the channel.
__device__ __forceinline__ void op_done(const XOp& X, uint64_t seq, bool sys) {
  __threadfence();  // this CTA's accesses to the ring are complete (their values were used)
  const uint32_t old = atomicAdd(X.done, 1u);
  if (old + 1 == (uint32_t)X.ncta) {
    atomicExch(X.done, 0u);
    *(volatile uint64_t*)X.seqp = seq;  // read by the next kernel on the stream
    __threadfence();
    if (X.role == 1) st_release(X.go, seq, sys);
  }
}

template <int NOPS>
__global__ void __launch_bounds__(kXferThreads, 1) k_xfer(const __grid_constant__ XArgsT<NOPS> A) {
  // dynamic smem: [staging buffers / record or span buffers] [word table]
  extern __shared__ __align__(128) uint8_t xsm[];
  __shared__ __align__(8) uint64_t mbar[kGroups][kXferStageBufs];
  uint8_t* sbuf = xsm;
  int32_t* wt = reinterpret_cast<int32_t*>(xsm + A.wt_off);
  __shared__ uint64_t s_n;
  __shared__ int s_stop, s_gs, s_rep;
  int op = 0;
  for (int i = 0; i < A.nops; i++)
    if ((int)blockIdx.x >= A.ops[i].cta0 && (int)blockIdx.x < A.ops[i].cta0 + A.ops[i].ncta) op = i;
  const XOp& X = A.ops[op];
  const int j = (int)blockIdx.x - X.cta0;
  const bool sleep_ok = !(A.flags & 2);
  // programmatic dependent launch (DT_XFER_PDL): the next transfer on the stream may start
  // its launch and setup now; it waits (griddepcontrol.wait below) before touching memory
  // this kernel or any earlier one writes.  (No-ops without PDL.)
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x == 0) xtrace(A, op, j, kTracePieces - 1, 0);  // (diagnostics: kernel entry)

  if (X.kind == 2 || X.kind == 4)
    for (int i = threadIdx.x; i < X.P.nwords; i += blockDim.x) wt[i] = X.P.wtab[i];
  if (X.kind == 6) {  // record-span maps after the per-warp buffers (same layout as xc_rec)
    const RecGeo& R = X.rg;
    uint16_t* omap = reinterpret_cast<uint16_t*>(xsm + kCopyWarps * (R.RB * R.spanB + R.RB * 8));
    if (X.role == 1) {
      switch (X.g) { case 4: rec_maps<true, 4>(R, omap); break; case 8: rec_maps<true, 8>(R, omap); break;
                     default: rec_maps<true, 16>(R, omap); break; }
    } else {
      switch (X.g) { case 4: rec_maps<false, 4>(R, omap); break; case 8: rec_maps<false, 8>(R, omap); break;
                     default: rec_maps<false, 16>(R, omap); break; }
    }
  }
  // prerequisite grids (the previous message's kernel, whatever produced the send buffer)
  // have completed and their memory is visible from here on
  asm volatile("griddepcontrol.wait;" ::: "memory");
  // every CTA of the op reads the same number: it is advanced only after all of them
  // have counted themselves done (op_done)
  const uint64_t seq = *(volatile const uint64_t*)X.seqp + 1;
  const bool sys = X.sys != 0;
  if (threadIdx.x == 0) {
    xtrace(A, op, j, kTracePieces - 1, 1);  // setup done
    uint64_t v = 0;
    s_stop = 0;
    if (X.role == 0) {
      // the receiver consumed the previous message on the channel: every slot is free
      const uint64_t prev = seq - 1;
      const bool ok = spin(X.go, [prev](uint64_t x) { return x >= prev; }, A.timeout_ns, X.err, &v, sleep_ok, sys);
      if (ok && j == 0) {
        st_relaxed(X.hdr + 1, (uint64_t)X.n, sys);
        st_relaxed(X.hdr + 2, (uint64_t)X.gs, sys);
        st_relaxed(X.hdr + 3, (uint64_t)X.rep, sys);
        st_release(X.hdr, seq, sys);
      }
      s_stop = !ok;
      s_n = (uint64_t)X.n;
      s_gs = X.gs;
      s_rep = X.rep;
    } else {
      const bool ok = spin(X.hdr, [seq](uint64_t x) { return x >= seq; }, A.timeout_ns, X.err, &v, sleep_ok, sys);
      const uint64_t nv = ok ? *(volatile uint64_t*)(X.hdr + 1) : 0;
      s_gs = ok ? (int)*(volatile uint64_t*)(X.hdr + 2) : 1;
      s_rep = ok ? (int)*(volatile uint64_t*)(X.hdr + 3) : 1;
      s_n = nv;
      const bool trunc = ok && nv > (uint64_t)X.n;
      s_stop = !ok || trunc;
      if (trunc && j == 0) {
        atomicCAS(X.err, 0, XERR_TRUNCATE);
        st_release(X.go + 1, seq, sys);  // aborted: a sender waiting for a slot stops
      }
    }
  }
  __syncthreads();
  if (s_stop) {
    if (threadIdx.x == 0) op_done(X, seq, sys);
    return;
  }
  const int64_t n = (int64_t)s_n;
  // Warp specialisation: warp 0 (lane 0) is the control warp -- it waits for each
  // piece's flag, hands the piece to the copy warps through full[b], waits for the
  // copy through empty[b] and publishes it -- so the flag latency and the release
  // (a system-scope release waits for every store of the piece to be acknowledged,
  // ~4 us over the system fabric) overlap the copy of the next piece.  Two pieces
  // in flight per CTA (b = piece index % 2).
  __shared__ __align__(8) uint64_t full[2], empty[2];
  __shared__ int s_abort;
  if (threadIdx.x == 0) {
    mbar_init(full + 0, 1);
    mbar_init(full + 1, 1);
    mbar_init(empty + 0, kGroupThreads);
    mbar_init(empty + 1, kGroupThreads);
    for (int g = 0; g < kGroups; g++)  // the staged unpack's TMA barriers: initialised once per kernel
      for (int b = 0; b < kXferStageBufs; b++) mbar_init(&mbar[g][b], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    s_abort = 0;
  }
  __syncthreads();
  if (threadIdx.x == 0) xtrace(A, op, j, kTracePieces - 1, 2);  // handshake done
  PieceIt it;
  bool more = it.init(X.role, n, X.chunk, X.depth, s_gs, s_rep, X.ncta, j);
  if (threadIdx.x < 32) {  // ---- control warp
    if (threadIdx.x != 0) return;
    // Event loop over two conditions, never blocking on one while the other could
    // progress (a receiver must publish piece i-1 before it can get piece i when the
    // sender has one slot per lane): release the oldest acquired piece once copied;
    // acquire the next piece when its flag is set (at most 2 pieces outstanding).
    int i_acq = 0, i_rel = 0;
    int q_fi[2] = {0, 0};
    uint64_t q_tag[2] = {0, 0};
    bool q_pub[2] = {true, true};
    uint64_t t_idle = 0;
    int ns = 0;
    while (more || i_rel < i_acq) {
      bool progress = false;
      if (i_rel < i_acq && mbar_test(empty + (i_rel & 1), (uint32_t)((i_rel >> 1) & 1))) {
        xtrace(A, op, j, i_rel, 2);
        if (A.flags & 4) __threadfence_system();
        const int b = i_rel & 1;
        if (q_pub[b]) st_release(X.role == 0 ? X.ready + q_fi[b] : X.ack + q_fi[b], q_tag[b], sys);
        xtrace(A, op, j, i_rel, 3);
        i_rel++;
        progress = true;
      }
      if (more && i_acq - i_rel < ((A.flags & 16) ? 1 : 2)) {
        const int fi = it.fi();
        const uint64_t tag = xtag(seq, it.round);
        bool ok;
        if (i_acq == 0 || ns == 0) xtrace(A, op, j, i_acq, 0);
        if (X.role == 0) ok = it.round == 0 || ld_acquire(X.ack + fi, sys) >= xtag(seq, it.round - 1);
        else ok = ld_acquire(X.ready + fi, sys) >= tag;
        if (ok) {
          xtrace(A, op, j, i_acq, 1);
          const int b = i_acq & 1;
          q_fi[b] = fi;
          q_tag[b] = tag;
          // an ack is read only by the same message's sender before it reuses the slot
          // (fragment k + D); the last D fragments' acks are dead (the next message
          // starts after "consumed", op_done) -- skipping them shortens a short message
          q_pub[b] = X.role == 0 || (A.flags & 64) || (int64_t)it.k + it.D < it.K;
          mbar_arrive(full + b);  // piece i_acq may be copied (the arrive releases the acquire)
          i_acq++;
          more = it.next();
          progress = true;
        }
      }
      if (progress) {
        t_idle = 0;
        ns = 0;
        continue;
      }
      // a sender waiting for a slot: has the receiver aborted the message (truncation)?
      if (X.role == 0 && i_rel == i_acq && ld_acquire(X.go + 1, sys) >= seq) {
        atomicCAS(X.err, 0, XERR_TRUNCATE);
        s_abort = 1;
        __threadfence_block();
        mbar_arrive(full + 0);
        mbar_arrive(full + 1);
        op_done(X, seq, sys);
        return;
      }
      if (sleep_ok) __nanosleep(ns);
      ns = ns < 16 ? 16 : (ns < 64 ? 2 * ns : 64);
      const uint64_t now = gtimer();
      if (!t_idle) t_idle = now;
      else if ((int64_t)(now - t_idle) > A.timeout_ns) {
        atomicCAS(X.err, 0, XERR_TIMEOUT);
        s_abort = 1;
        __threadfence_block();
        // wake both copy groups (each waits on its own barrier); they see s_abort and leave.
        // A group still copying its piece leaves at its next wait: that phase completes by
        // these arrivals or by the one below.
        mbar_arrive(full + 0);
        mbar_arrive(full + 1);
        op_done(X, seq, sys);
        return;
      }
    }
    xtrace(A, op, j, kTracePieces - 1, 3);  // control loop done
    op_done(X, seq, sys);
    return;
  }
  // ---- copy groups: group g takes the CTA's pieces g, g + 2, g + 4, ...
  const int g = (threadIdx.x - 32) / kGroupThreads;
  int64_t tb = 0;  // tiles this group has moved through its TMA barriers (staged unpack)
  if (more && g == 1) more = it.next();
  for (int i = g; more; i += 2) {
    mbar_wait(full + g, (uint32_t)((i >> 1) & 1));
    if (s_abort) return;
    const int64_t off = it.off();
    uint8_t* sl = X.ring + (int64_t)it.slot * X.chunk + (int64_t)it.js * it.Cs - off;  // stream byte off -> piece
    // the staged (4) and block-span (7) unpacks read the ring slot with TMA bulk loads
    // (async proxy): order them after the control warp's generic-proxy acquire
    if (X.role == 1 && (X.kind == 4 || X.kind == 7) && !(A.flags & 8))
      asm volatile("fence.proxy.async.global;" ::: "memory");
    if (threadIdx.x == 32 + g * kGroupThreads) xtrace(A, op, j, i, 4);
    if (X.role == 0) cta_piece<false>(X, sl, off, it.len(), wt, sbuf, mbar[g], g, tb);
    else cta_piece<true>(X, sl, off, it.len(), wt, sbuf, mbar[g], g, tb);
    if (threadIdx.x == 32 + g * kGroupThreads) xtrace(A, op, j, i, 5);
    mbar_arrive(empty + g);  // release.cta: this thread's stores precede the control warp's wait
    more = it.next() && it.next();
  }
}

// ------------------------------------------------------------------ copy-engine mode
// DT_XFER_CE: the paper's receiver staging with the copy engine as the wire
// ([L20:c4255 §4.1]): the sender packs each fragment into a local staging
// slot (a pack kernel), the copy engine moves it into the receiver's ring slot
// (cudaMemcpyAsync to the IPC-mapped peer address), and stream-ordered one-thread
// kernels publish / await the same tag flags the P2P kernel uses.  Host-driven: every
// fragment is a few stream operations on three internal streams.
__global__ void k_ce_wait(const uint64_t* __restrict__ p, uint64_t v, int sys, int64_t timeout_ns, int32_t* err) {
  if (threadIdx.x != 0) return;
  const uint64_t t0 = gtimer();
  while (ld_acquire(p, sys != 0) < v) {
    __nanosleep(64);
    if ((int64_t)(gtimer() - t0) > timeout_ns) {
      atomicCAS(err, 0, XERR_TIMEOUT);
      return;
    }
  }
}
// p[1..nx] = x[0..nx) (relaxed), then p[0] = v (release)
__global__ void k_ce_signal(uint64_t* p, uint64_t v, int sys, uint64_t x0, int nx) {
  if (threadIdx.x != 0) return;
  if (nx > 0) p[1] = x0;
  st_release(p, v, sys != 0);
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
  int32_t mode;
  int64_t chunk_bytes;  // the ring geometry every peer must share (checked at connect)
  int32_t depth, nch;
  uint8_t uuid[16];     // physical GPU (device ordinals differ between processes)
  uint64_t ring_ptr, flags_ptr;
  cudaIpcMemHandle_t ring_h, flags_h;
};
static const uint32_t kMagic = 0xD7A7C0E2u;

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
  size_t ring_bytes = 0, flag_words = 0;
  std::vector<uint8_t*> peer_ring;
  std::vector<uint64_t*> peer_flags;
  std::vector<bool> opened;
  std::vector<int> same_dev;  // peer runs on this physical GPU: gpu-scope flags suffice
  bool connected = false;
  // device-resident per-(role, peer, channel) sequence numbers and CTA counters (local)
  uint64_t* dseq = nullptr;   // [2][nranks][nch]
  uint32_t* ddone = nullptr;  // [2][nranks][nch]
  // group
  bool in_group = false;
  std::vector<PendingOp> pending;
  // CE mode: host sequence numbers per (role, peer, channel) and the last tag published
  // into each of a peer's ring slots (a slot is reused once its ack has reached that tag)
  std::vector<uint64_t> hseq;
  std::vector<uint64_t> slot_tag;  // [nranks][nch][depth]
  // NCCL mode
  ncclComm_t nccl = nullptr;
  cudaStream_t s_pack = nullptr, s_net = nullptr, s_unpack = nullptr;
  std::vector<cudaEvent_t> ev;
  uint8_t* stage = nullptr;  // send staging [kMaxOps][depth][chunk]
  uint8_t* rstage = nullptr; // recv staging
  int64_t* szbuf = nullptr;  // device size handshake buffers [2][kMaxOps]
  int64_t* szhost = nullptr; // pinned
  // layout helpers (uint64 flag words): per (peer, channel) depth*kMaxSub ready tags,
  // a 4-word header {seq, nbytes|abort, pieces, teams}, depth*kMaxSub ack tags and
  // a 2-word go {consumed seq, aborted seq}, a receiver-local CTA counter; then one
  // error word.  The ring of a (source,
  // channel) pair is depth*chunk bytes: D slots of one fragment each.
  size_t per() const { return (size_t)kMaxSub * o.depth; }
  size_t pairs() const { return (size_t)nranks * nch; }
  size_t ready_idx(int src, int ch) const { return ((size_t)src * nch + ch) * per(); }
  size_t hdr_idx(int src, int ch) const { return pairs() * per() + ((size_t)src * nch + ch) * 4; }
  size_t ack_idx(int dst, int ch) const { return pairs() * (per() + 4) + ((size_t)dst * nch + ch) * per(); }
  size_t go_idx(int dst, int ch) const { return pairs() * (2 * per() + 4) + ((size_t)dst * nch + ch) * 2; }
  size_t done_idx(int src, int ch) const { return pairs() * (2 * per() + 6) + (size_t)src * nch + ch; }
  size_t err_idx() const { return pairs() * (2 * per() + 7); }
  size_t ring_off(int src, int ch) const { return (((size_t)src * nch + ch) * o.depth) * (size_t)o.chunk_bytes; }
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
  o.depth = 0;
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
  // a fragment is a ring slot: <= 1 GiB (the transfer kernel's piece arithmetic is 32-bit
  // within a fragment)
  o.chunk_bytes = std::min<int64_t>(o.chunk_bytes, int64_t(1) << 30);
  if ((!in || in->depth <= 0) && o.mode == DT_XFER_NCCL) {
    o.depth = 4;  // NCCL mode: depth = staging buffers of the pack/net/unpack overlap
  } else if (!in || in->depth <= 0) {
    // auto depth: a ring of >= 8 MiB per (pair, channel), at least 4 slots -- the
    // in-flight bytes must cover link bandwidth x flag round trip (900 GB/s x ~5 us),
    // so small fragments need many slots (64 KiB: 128)
    int64_t d = ((int64_t)8 << 20) / o.chunk_bytes;
    o.depth = (int)std::max<int64_t>(4, std::min<int64_t>(kMaxDepth, d));
  }
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
  if (c->o.mode != DT_XFER_P2P && c->o.mode != DT_XFER_NCCL && c->o.mode != DT_XFER_CE) {
    delete c;
    set_error("dt_comm_init: unknown mode");
    return DT_ERR_ARG;
  }
  if (c->o.depth > kMaxDepth) {
    delete c;
    set_error("dt_comm_init: depth %d > %d", c->o.depth, kMaxDepth);
    return DT_ERR_ARG;
  }
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) {
    delete c;
    return cufail(e, "cudaSetDevice");
  }
  c->ring_bytes = (size_t)nranks * c->nch * c->o.depth * (size_t)c->o.chunk_bytes;
  c->flag_words = c->err_idx() + 1;
  if (c->o.mode == DT_XFER_P2P || c->o.mode == DT_XFER_CE) {
    e = cudaMalloc(&c->ring, c->ring_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&c->flags, c->flag_words * 8);
    if (e == cudaSuccess) e = cudaMemset(c->flags, 0, c->flag_words * 8);
    const size_t nq = (size_t)2 * nranks * c->nch;
    if (e == cudaSuccess) e = cudaMalloc(&c->dseq, nq * 8);
    if (e == cudaSuccess) e = cudaMemset(c->dseq, 0, nq * 8);
    if (e == cudaSuccess) e = cudaMalloc(&c->ddone, nq * 4);
    if (e == cudaSuccess) e = cudaMemset(c->ddone, 0, nq * 4);
    if (e != cudaSuccess) {
      cudaFree(c->ring);
      cudaFree(c->flags);
      cudaFree(c->dseq);
      cudaFree(c->ddone);
      delete c;
      return cufail(e, "dt_comm_init alloc");
    }
    if (c->o.mode == DT_XFER_CE) {
      const size_t st = (size_t)kMaxOps * c->o.depth * (size_t)c->o.chunk_bytes;
      e = cudaMalloc(&c->stage, st);
      if (e == cudaSuccess) e = cudaMalloc(&c->szbuf, sizeof(int64_t) * 2 * kMaxOps);
      if (e == cudaSuccess) e = cudaMallocHost(&c->szhost, sizeof(int64_t) * 2 * kMaxOps);
      if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s_pack, cudaStreamNonBlocking);
      if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s_net, cudaStreamNonBlocking);
      if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s_unpack, cudaStreamNonBlocking);
      if (e != cudaSuccess) return cufail(e, "dt_comm_init ce alloc");
      c->ev.resize((size_t)kMaxOps * c->o.depth * 3 + 2);
      for (auto& x : c->ev) cudaEventCreateWithFlags(&x, cudaEventDisableTiming);
      c->hseq.assign((size_t)2 * nranks * c->nch, 0);
      c->slot_tag.assign((size_t)nranks * c->nch * c->o.depth, 0);
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
  c->same_dev.assign(nranks, 0);
  c->same_dev[rank] = !getenv("DT_XFER_SYS");  // DT_XFER_SYS: system-scope flags even on one GPU

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
  b.mode = c->o.mode;
  b.chunk_bytes = c->o.chunk_bytes;
  b.depth = c->o.depth;
  b.nch = c->nch;
  {
    cudaDeviceProp pr;
    CU(cudaGetDeviceProperties(&pr, c->device));
    std::memcpy(b.uuid, &pr.uuid, 16);
  }
  b.ring_ptr = (uint64_t)(uintptr_t)c->ring;
  b.flags_ptr = (uint64_t)(uintptr_t)c->flags;
  if (c->o.mode == DT_XFER_P2P || c->o.mode == DT_XFER_CE) {
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
  if (c->o.mode == DT_XFER_NCCL) {
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
    if (b.mode != c->o.mode || b.chunk_bytes != c->o.chunk_bytes || b.depth != c->o.depth || b.nch != c->nch) {
      // the sender lays fragments out with its own C and D inside the receiver's ring
      set_error("dt_comm_connect: rank %d uses chunk %lld / depth %d / mode %d, this rank chunk %lld / depth %d / "
                "mode %d (must match)", r, (long long)b.chunk_bytes, b.depth, b.mode, (long long)c->o.chunk_bytes,
                c->o.depth, c->o.mode);
      return DT_ERR_ARG;
    }
    if (r == c->rank) continue;
    {
      cudaDeviceProp pr;
      CU(cudaGetDeviceProperties(&pr, c->device));
      c->same_dev[r] = std::memcmp(b.uuid, &pr.uuid, 16) == 0 && !getenv("DT_XFER_SYS");
    }
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
// Contiguous instances are merged into one run first (effective(): count BYTEs, a
// vector of adjacent blocks), so a piece of a contiguous message is one warp copy
// per warp slice instead of a walk over count tiny instances.
static dt_status side_params(dt_t t, int64_t count, const void* nc, int64_t nbytes, int64_t chunk, XOp& X) {
  DeviceDesc* dd = nullptr;
  dt_status st = ensure_committed_on_device(t, &dd);
  if (st != DT_OK) return st;
  const Form& f = get_form(t);
  const Eff E = effective(f, dd, t, count);
  const KLevels& L = E.L;
  KP& P = X.P;
  std::memset(&P, 0, sizeof(P));
  P.nc = (const uint8_t*)nc;
  P.tsize = E.tsize;
  P.nblocks = E.nblocks;
  P.bd = dd->bd;
  P.bl = dd->bl;
  P.boff = dd->boff;
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
  // piece starts are multiples of C/gs (a multiple of 512) and ring slots are aligned
  int kind = E.merged ? 1 : plan_kernel(f, L, (uint64_t)(uintptr_t)nc, 0, 0, nbytes, &g);
  if (kind == 6) {  // record spans: pieces start on 512-byte stream boundaries (16-byte aligned)
    if (!rec_geometry(f, L, (uint64_t)(uintptr_t)nc, 0, 0, nbytes, g, &X.rg) || getenv("DT_XFER_NOREC"))
      kind = g >= stage_min_g() ? 4 : 2;
  }
  if ((kind == 2 || kind == 4 || kind == 6 || kind == 7) && lowp2u((uint64_t)chunk) < g) kind = 1;
  if (kind == 4 && g < std::max<int64_t>(4, stage_min_g())) kind = 2;
  if (kind == 2 && g >= std::max<int64_t>(4, stage_min_g()) && !getenv("DT_XFER_NOSTAGE")) kind = 4;
  if (kind == 7 && getenv("DT_XFER_NOSPAN")) kind = 1;
  // the block-window kernel (3) is not used inside the pipeline
  X.kind = (kind == 2 || kind == 4 || kind == 6 || kind == 7) ? kind : 1;
  if (const char* fk = getenv("DT_XFER_KIND")) {  // tuning: force a family where it applies
    const int k = atoi(fk);
    const bool wt_ok = f.tsize() / g <= kMaxWordTable && f.tsize() % g == 0 && !E.merged;
    if ((k == 2 && wt_ok) || (k == 4 && wt_ok && g >= 4) || k == 1) X.kind = k;
  }
  if (X.kind == 7) {
    P.fnb = make_fd((uint64_t)P.nblocks);
    st = ensure_sdesc(f, *dd, &P.sdesc, &P.wbase);
    if (st != DT_OK) return st;
  }
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
// displacements, then the per-CTA map (layout as in xc_rec / k_xfer)
static size_t rec_smem_bytes(const RecGeo& R, int g) {
  const size_t nwc = kCopyWarps;
  const size_t tab = std::max<size_t>((size_t)R.RB * R.nwr * 2, (size_t)(R.spanB / g) * 2);
  return nwc * ((size_t)R.RB * R.spanB + (size_t)R.RB * 8) + tab;
}

// CTA budget per direction (capped by co-residency across the group's ops)
static int default_ctas(const dt_comm_s* c) {
  if (c->o.ctas > 0) return c->o.ctas;
  const char* e = getenv("DT_XFER_CTAS");
  return e && atoi(e) > 0 ? atoi(e) : 64;
}

// Message geometry (gs pieces per fragment, rep teams): pieces of >= kPiece bytes
// (a CTA moves a piece with one barrier + one flag; smaller pieces are all fixed
// cost), as many pieces as the budget allows for large fragments, then teams that
// take alternate fragments so several fragments are in flight at once (each team
// owns D/rep slots).  Depends only on (n, C, D, budget).
struct Geo {
  int gs, gu, rep;
};
static Geo geometry(int64_t n, int64_t C, int D, int budget, double w = 1.0) {
  static const int64_t kPiece0 = getenv("DT_XFER_PIECE") ? atoll(getenv("DT_XFER_PIECE")) : (32 << 10);
  // a family that moves bytes w times slower per CTA amortises the per-piece fixed cost
  // (flag release, barriers) over w times fewer bytes
  int64_t kPiece = std::max<int64_t>(4096, (int64_t)(kPiece0 / std::max(1.0, w)));
  // a message of one fragment is latency-bound: spread it over up to the budget's CTAs in
  // pieces of >= 4 KiB (a piece's fixed costs overlap across CTAs instead of adding up)
  if (n > C) kPiece = kPiece0;  // (several fragments: teams on alternate fragments matter more)
  else if (!getenv("DT_XFER_PIECE")) kPiece = std::min(kPiece, std::max<int64_t>(4096, n / std::max(1, budget)));
  const int64_t eff = std::min<int64_t>(C, std::max<int64_t>(512, (n + 511) & ~int64_t(511)));
  // p: pieces per fragment, >= kPiece bytes each, up to two per CTA of the budget (a
  // CTA's two copy groups take alternate pieces: with one piece per CTA -- a message of
  // one fragment -- the second group would idle)
  int p = 1;
  // (one fragment: as many pieces as the slot layout allows, several per CTA, so the
  // receiver starts on the first pieces while the sender packs the later ones -- the
  // paper's pipeline inside one fragment)
  while (p * 2 <= kMaxSub && (n <= C || p * 2 <= 2 * budget) && eff / (p * 2) >= kPiece) p *= 2;
  // gs: the slot layout, pieces of C/gs >= eff/p bytes (a message shorter than C uses
  // gu < gs of them)
  const int64_t want = (((eff + p - 1) / p) + 511) & ~int64_t(511);
  int gs = 1;
  while (gs * 2 <= kMaxSub && C % ((int64_t)gs * 2 * 512) == 0 && C / (gs * 2) >= want) gs *= 2;
  const int64_t Cs = C / gs;
  const int gu = (int)std::max<int64_t>(1, std::min<int64_t>(gs, (std::min(n, C) + Cs - 1) / Cs));
  const int64_t K = std::max<int64_t>(1, (n + C - 1) / C);
  const char* rp = getenv("DT_XFER_REP");
  int rep = 1;
  if (rp) {
    rep = std::max(1, atoi(rp));
    while (rep > 1 && (D % rep || rep * gu > budget)) rep--;
  } else {
    while (rep * 2 <= D && D % (rep * 2) == 0 && rep * 2 * gu <= budget && rep * 2 <= K) rep *= 2;
  }
  return Geo{gs, gu, rep};
}

static dt_status issue_p2p(dt_comm_s* c, const std::vector<PendingOp>& ops, cudaStream_t s) {
  XArgs A;
  std::memset(&A, 0, sizeof(A));
  const char* to = getenv("DT_TIMEOUT_MS");
  A.timeout_ns = (int64_t)(to ? atoll(to) : 30000) * 1000000ll;
  A.flags = getenv("DT_XFER_FLAGS") ? atoi(getenv("DT_XFER_FLAGS")) : 0;
  int nops = 0;
  size_t smem = 0, rec_smem = 0;
  bool any_stage = false;
  std::vector<int> sch(c->nranks, 0), rch(c->nranks, 0);
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
      uint64_t* pf = c->peer_flags[p.dest];
      X.ring = c->peer_ring[p.dest] + c->ring_off(c->rank, ch);
      X.ready = pf + c->ready_idx(c->rank, ch);
      X.hdr = pf + c->hdr_idx(c->rank, ch);
      X.ack = c->flags + c->ack_idx(p.dest, ch);
      X.go = c->flags + c->go_idx(p.dest, ch);
      X.seqp = c->dseq + ((size_t)0 * c->nranks + p.dest) * c->nch + ch;
      X.done = c->ddone + ((size_t)0 * c->nranks + p.dest) * c->nch + ch;
      X.sys = !c->same_dev[p.dest];
      // a peer on another GPU: the staged family's tiles leave with plain coalesced
      // 16-byte stores (no TMA bulk stores into peer memory, never exercised on a
      // one-GPU lease; X.sys selects them in xc_stage)
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
      uint64_t* pf = c->peer_flags[p.source];
      X.ring = c->ring + c->ring_off(p.source, ch);
      X.ready = c->flags + c->ready_idx(p.source, ch);
      X.hdr = c->flags + c->hdr_idx(p.source, ch);
      X.ack = pf + c->ack_idx(c->rank, ch);
      X.go = pf + c->go_idx(c->rank, ch);
      X.seqp = c->dseq + ((size_t)1 * c->nranks + p.source) * c->nch + ch;
      X.done = c->ddone + ((size_t)1 * c->nranks + p.source) * c->nch + ch;
      X.sys = !c->same_dev[p.source];
    }
  }
  if (nops == 0) return DT_OK;
  for (int i = 0; i < nops; i++) {
    XOp& X = A.ops[i];
    X.chunk = c->o.chunk_bytes;
    X.depth = c->o.depth;
    X.err = reinterpret_cast<int32_t*>(c->flags + c->err_idx());
    if (X.kind == 2 || X.kind == 4) smem = std::max(smem, sizeof(int32_t) * (size_t)X.P.nwords);
    any_stage = any_stage || X.kind == 4;
    if (X.kind == 6) rec_smem = std::max(rec_smem, rec_smem_bytes(X.rg, X.g));
    if (X.kind == 7) rec_smem = std::max(rec_smem, (size_t)kCopyWarps * kSpanWarpSmem);
  }
  A.nops = nops;
  A.wt_off = (int32_t)std::max<size_t>(any_stage ? (size_t)kGroups * kXferStageBufs * kStageTile : 0,
                                       (rec_smem + 127) & ~size_t(127));
  smem += (size_t)A.wt_off;
  // the attribute is per device (a process may drive several)
  const void* kfn = nops <= 2 ? (const void*)k_xfer<2> : (const void*)k_xfer<kMaxOps>;
  if (smem > 48 * 1024) CU(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  // every CTA must be co-resident: fit the per-op CTA budget to the occupancy
  int occ = 0;
  CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kfn, kXferThreads, smem));
  int sms = 0, dev = 0;
  CU(cudaGetDevice(&dev));
  CU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  // Co-resident CTAs are shared among the ops in proportion to their estimated cost:
  // bytes x a per-family factor (4-byte words gathered one by one cost ~4x a long-run
  // copy per byte; the C4 halo's x faces next to its y/z faces).
  // Unpacking G-byte words scatters partial-sector writes (each a DRAM read-modify-write
  // when G < 32): measured ~2x the pack cost, so the factor doubles on the receive side.
  auto cost = [](const XOp& X) {
    double w = (X.kind == 2 || X.kind == 4) ? 16.0 / X.g : (X.kind == 6 || X.kind == 7) ? 2.0 : 1.0;
    if (X.role == 1 && X.g < 16 && X.kind != 1) w *= 2;
    return (double)std::max<int64_t>(X.n, 4096) * w;
  };
  double csum = 0;
  for (int i = 0; i < nops; i++) csum += cost(A.ops[i]);
  const int total = occ * sms;
  // every op gets the default budget when all of them fit; otherwise shares by cost
  const bool fits = (int64_t)nops * default_ctas(c) <= total;
  int cta = 0;
  int np[kMaxOps], ppc[kMaxOps];
  for (int i = 0; i < nops; i++) {
    XOp& X = A.ops[i];
    const int budget = fits ? default_ctas(c)
                            : std::max(1, std::min(default_ctas(c), (int)(total * cost(X) / csum)));
    // send role: one CTA per (team, piece); receive role: as many as the capacity
    // would need (the actual geometry arrives in the header; CTAs map onto it)
    const Geo G = geometry(X.n, X.chunk, X.depth, budget, cost(X) / (double)std::max<int64_t>(X.n, 4096));
    X.gs = G.gs;
    X.rep = G.rep;
    // pairs (team, piece) beyond the budget: CTAs take several (pairs j, j + ncta, ...)
    np[i] = G.gu * G.rep;
    ppc[i] = (np[i] + budget - 1) / budget;
    X.ncta = (np[i] + ppc[i] - 1) / ppc[i];
    cta += X.ncta;
  }
  // Co-resident CTAs the shares left unused (budgets round down to whole pieces per CTA):
  // give them to the op whose CTAs carry the most work (cost per piece x pieces per CTA)
  // while the next step fits -- the group's makespan is its slowest op's.
  while (!fits) {
    int best = -1;
    double bt = -1;
    for (int i = 0; i < nops; i++) {
      const double t = cost(A.ops[i]) / np[i] * ppc[i];
      if (t > bt) { bt = t; best = i; }
    }
    if (best < 0 || ppc[best] <= 1) break;
    const int nn = (np[best] + ppc[best] - 2) / (ppc[best] - 1);
    if (cta - A.ops[best].ncta + nn > total) break;
    cta += nn - A.ops[best].ncta;
    A.ops[best].ncta = nn;
    ppc[best]--;
  }
  cta = 0;
  for (int i = 0; i < nops; i++) {
    A.ops[i].cta0 = cta;
    cta += A.ops[i].ncta;
  }
  if (getenv("DT_XFER_DEBUG"))
    for (int i = 0; i < nops; i++)
      fprintf(stderr, "[dt_xfer] op %d role %d kind %d g %d n %lld C %lld D %d gs %d rep %d ncta %d total %d\n", i,
              A.ops[i].role, A.ops[i].kind, A.ops[i].g, (long long)A.ops[i].n, (long long)A.ops[i].chunk,
              A.ops[i].depth, A.ops[i].gs, A.ops[i].rep, A.ops[i].ncta, total);
  static uint64_t* trace = nullptr;
  const char* tr = getenv("DT_XFER_TRACE");  // diagnostics: dump per-piece timestamps to this file
  const size_t tn = (size_t)kMaxOps * kTraceCtas * kTracePieces * kTracePts;
  if (tr) {  // host-mapped, so a hung kernel's progress is readable
    if (!trace) CU(cudaHostAlloc(&trace, tn * 8, cudaHostAllocMapped));
    CU(cudaStreamSynchronize(s));
    std::memset(trace, 0, tn * 8);
    A.trace = trace;
  }
  // every CTA of both roles must be co-resident (they wait on each other): cooperative launch
  void* args[] = {&A};
  static const bool coop = !getenv("DT_XFER_NOCOOP");
  XArgsT<2> A2;  // a single exchange: the small parameter block
  if (nops <= 2) {
    std::memcpy(&A2, &A, offsetof(XArgs, ops));
    std::memcpy(A2.ops, A.ops, sizeof(XOp) * 2);
    args[0] = &A2;
  }
  // DT_XFER_PDL=1: a plain launch with programmatic stream serialisation, so back-to-back
  // transfers overlap the next kernel's launch and setup with the current one (the grid is
  // sized to fit co-resident, as for DT_XFER_NOCOOP; no cooperative guarantee);
  // DT_XFER_PDL=2: cooperative as well
  static const bool pdl = getenv("DT_XFER_PDL") && atoi(getenv("DT_XFER_PDL")) > 0;
  if (pdl) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(cta);
    cfg.blockDim = dim3(kXferThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    at[1].id = cudaLaunchAttributeCooperative;  // DT_XFER_PDL=2: keep the co-residency guarantee too
    at[1].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = atoi(getenv("DT_XFER_PDL")) >= 2 && coop ? 2 : 1;
    CU(cudaLaunchKernelExC(&cfg, kfn, args));
  } else if (coop) {
    CU(cudaLaunchCooperativeKernel(kfn, dim3(cta), dim3(kXferThreads), args, smem, s));
  } else {
    CU(cudaLaunchKernel(kfn, dim3(cta), dim3(kXferThreads), args, smem, s));
  }
  if (tr) {
    bool hung = false;
    for (int w = 0; cudaStreamQuery(s) == cudaErrorNotReady; w++) {
      if (w > 5000) { hung = true; break; }  // ~5 s
      usleep(1000);
    }
    if (FILE* fp = fopen(tr, "a")) {
      fprintf(fp, "# launch nops %d%s\n", nops, hung ? " HUNG" : "");
      for (int i = 0; i < nops; i++)
        for (int jj = 0; jj < kTraceCtas; jj++)
          for (int p = 0; p < kTracePieces; p++) {
            const volatile uint64_t* q = &trace[(((size_t)i * kTraceCtas + jj) * kTracePieces + p) * kTracePts];
            if (q[0] || q[4]) {
              fprintf(fp, "%d %d %d %d", i, A.ops[i].role, jj, p);
              for (int k = 0; k < kTracePts; k++) fprintf(fp, " %llu", (unsigned long long)q[k]);
              fprintf(fp, "\n");
            }
          }
      fclose(fp);
    }
    if (hung) {
      fprintf(stderr, "[dt_xfer] kernel hung; trace written to %s\n", tr);
      _exit(3);
    }
  }
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

// Copy-engine mode (DT_XFER_CE, see k_ce_wait): per message a header {seq, n} in the
// receiver's flags (the receiver's host reads n: its unpack launches need the fragment
// lengths), then per fragment k (slot k % D): sender -- pack into its staging slot
// (s_pack), wait until the receiver acked the slot's previous tag, copy-engine copy into
// the receiver's ring slot and publish the ready tag (s_net); receiver -- wait for the
// ready tag, unpack from its ring slot, publish the ack tag into the sender's flags
// (s_unpack).  Tags are the P2P kernel's (seq, round) tags; a slot's first piece word
// carries them.
static dt_status issue_ce(dt_comm_s* c, const std::vector<PendingOp>& ops, cudaStream_t s) {
  const int64_t C = c->o.chunk_bytes;
  const int D = c->o.depth;
  struct Side { const PendingOp* p; int peer, ch; uint64_t seq; int64_t n; };
  std::vector<Side> sends, recvs;
  std::vector<int> sch(c->nranks, 0), rch(c->nranks, 0);
  for (const auto& p : ops) {
    if (p.dest >= 0) {
      const int ch = sch[p.dest]++;
      if (ch >= c->nch) { set_error("dt_sendrecv: more than %d messages to one peer in a group", c->nch); return DT_ERR_UNSUPPORTED; }
      uint64_t& q = c->hseq[((size_t)0 * c->nranks + p.dest) * c->nch + ch];
      sends.push_back({&p, p.dest, ch, ++q, p.scount * p.stype->size});
    }
    if (p.source >= 0) {
      const int ch = rch[p.source]++;
      if (ch >= c->nch) { set_error("dt_sendrecv: more than %d messages from one peer in a group", c->nch); return DT_ERR_UNSUPPORTED; }
      uint64_t& q = c->hseq[((size_t)1 * c->nranks + p.source) * c->nch + ch];
      recvs.push_back({&p, p.source, ch, ++q, 0});
    }
  }
  if ((int)sends.size() > kMaxOps || (int)recvs.size() > kMaxOps) {
    set_error("dt_sendrecv: too many ops in one group");
    return DT_ERR_UNSUPPORTED;
  }
  const char* to = getenv("DT_TIMEOUT_MS");
  const int64_t tmo = (int64_t)(to ? atoll(to) : 30000) * 1000000ll;
  int32_t* err = reinterpret_cast<int32_t*>(c->flags + c->err_idx());
  cudaEvent_t* ev = c->ev.data();
  cudaEvent_t ev_start = ev[(size_t)kMaxOps * D * 3], ev_end = ev[(size_t)kMaxOps * D * 3 + 1];
  CU(cudaEventRecord(ev_start, s));
  CU(cudaStreamWaitEvent(c->s_pack, ev_start, 0));
  CU(cudaStreamWaitEvent(c->s_net, ev_start, 0));
  CU(cudaStreamWaitEvent(c->s_unpack, ev_start, 0));
  // headers first (a loopback receiver below waits for them on the host)
  for (const Side& x : sends) {
    uint64_t* hdr = c->peer_flags[x.peer] + c->hdr_idx(c->rank, x.ch);
    k_ce_signal<<<1, 32, 0, c->s_net>>>(hdr, x.seq, !c->same_dev[x.peer], (uint64_t)x.n, 1);
  }
  CU(cudaGetLastError());
  for (size_t i = 0; i < recvs.size(); i++) {
    const Side& x = recvs[i];
    const uint64_t* hdr = c->flags + c->hdr_idx(x.peer, x.ch);
    k_ce_wait<<<1, 32, 0, c->s_unpack>>>(hdr, x.seq, !c->same_dev[x.peer], tmo, err);
    CU(cudaMemcpyAsync(c->szhost + kMaxOps + i, hdr + 1, sizeof(int64_t), cudaMemcpyDeviceToHost, c->s_unpack));
  }
  CU(cudaGetLastError());
  if (!recvs.empty()) CU(cudaStreamSynchronize(c->s_unpack));
  for (size_t i = 0; i < recvs.size(); i++) {
    recvs[i].n = c->szhost[kMaxOps + i];
    const int64_t cap = recvs[i].p->rcount * recvs[i].p->rtype->size;
    if (recvs[i].n > cap) {
      // consume the message without unpacking it: ack every fragment with its final tag
      const int64_t K = (recvs[i].n + C - 1) / C;
      for (int64_t k = std::max<int64_t>(0, K - D); k < K; k++)
        k_ce_signal<<<1, 32, 0, c->s_unpack>>>(c->peer_flags[recvs[i].peer] + c->ack_idx(c->rank, recvs[i].ch) +
                                                   (size_t)(k % D) * kMaxSub,
                                               xtag(recvs[i].seq, k / D), !c->same_dev[recvs[i].peer], 0, 0);
      set_error("dt_sendrecv: message of %lld bytes truncated by a %lld-byte receive", (long long)recvs[i].n,
                (long long)cap);
      recvs[i].n = -1;
    }
  }
  bool trunc = false;
  for (const Side& x : recvs) trunc = trunc || x.n < 0;
  int64_t K = 0;
  for (const Side& x : sends) K = std::max(K, (x.n + C - 1) / C);
  for (const Side& x : recvs) K = std::max(K, (x.n + C - 1) / C);
  const size_t slot_span = (size_t)kMaxOps * C;
  auto ev_packed = [&](size_t i, int slot) { return ev[(i * D + slot) * 3]; };
  auto ev_sent = [&](size_t i, int slot) { return ev[(i * D + slot) * 3 + 1]; };
  for (int64_t k = 0; k < K; k++) {
    const int slot = (int)(k % D);
    const int64_t round = k / D;
    for (size_t i = 0; i < sends.size(); i++) {
      const Side& x = sends[i];
      int64_t pos = k * C, len = std::min<int64_t>(C, x.n - pos);
      if (len <= 0) continue;
      uint8_t* st_slot = c->stage + slot * slot_span + i * C;
      if (k >= D) CU(cudaStreamWaitEvent(c->s_pack, ev_sent(i, slot), 0));  // staging slot copied out
      dt_status st = dt_pack(x.p->stype, x.p->scount, x.p->sbuf, st_slot, pos, &len, c->s_pack);
      if (st != DT_OK) return st;
      CU(cudaEventRecord(ev_packed(i, slot), c->s_pack));
      CU(cudaStreamWaitEvent(c->s_net, ev_packed(i, slot), 0));
      // the receiver's ring slot is free once it acked the last tag published into it
      uint64_t& last = c->slot_tag[((size_t)x.peer * c->nch + x.ch) * D + slot];
      const bool sys = !c->same_dev[x.peer];
      if (last) k_ce_wait<<<1, 32, 0, c->s_net>>>(c->flags + c->ack_idx(x.peer, x.ch) + (size_t)slot * kMaxSub, last,
                                                   sys, tmo, err);
      uint8_t* dst = c->peer_ring[x.peer] + c->ring_off(c->rank, x.ch) + (size_t)slot * C;
      CU(cudaMemcpyAsync(dst, st_slot, (size_t)len, cudaMemcpyDeviceToDevice, c->s_net));
      last = xtag(x.seq, round);
      k_ce_signal<<<1, 32, 0, c->s_net>>>(c->peer_flags[x.peer] + c->ready_idx(c->rank, x.ch) + (size_t)slot * kMaxSub,
                                          last, sys, 0, 0);
      CU(cudaGetLastError());
      CU(cudaEventRecord(ev_sent(i, slot), c->s_net));
    }
    for (size_t i = 0; i < recvs.size(); i++) {
      const Side& x = recvs[i];
      int64_t pos = k * C, len = std::min<int64_t>(C, x.n - pos);
      if (x.n < 0 || len <= 0) continue;
      const bool sys = !c->same_dev[x.peer];
      k_ce_wait<<<1, 32, 0, c->s_unpack>>>(c->flags + c->ready_idx(x.peer, x.ch) + (size_t)slot * kMaxSub,
                                           xtag(x.seq, round), sys, tmo, err);
      dt_status st = dt_unpack(x.p->rtype, x.p->rcount, c->ring + c->ring_off(x.peer, x.ch) + (size_t)slot * C,
                               x.p->rbuf, pos, &len, c->s_unpack);
      if (st != DT_OK) return st;
      k_ce_signal<<<1, 32, 0, c->s_unpack>>>(c->peer_flags[x.peer] + c->ack_idx(c->rank, x.ch) + (size_t)slot * kMaxSub,
                                             xtag(x.seq, round), sys, 0, 0);
      CU(cudaGetLastError());
    }
  }
  CU(cudaEventRecord(ev_end, c->s_pack));
  CU(cudaStreamWaitEvent(s, ev_end, 0));
  CU(cudaEventRecord(ev_end, c->s_net));
  CU(cudaStreamWaitEvent(s, ev_end, 0));
  CU(cudaEventRecord(ev_end, c->s_unpack));
  CU(cudaStreamWaitEvent(s, ev_end, 0));
  return trunc ? DT_ERR_TRUNCATE : DT_OK;
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
  if (c->o.mode == DT_XFER_CE) return issue_ce(c, ops_in, s);
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
  cudaFree(c->dseq);
  cudaFree(c->ddone);
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
