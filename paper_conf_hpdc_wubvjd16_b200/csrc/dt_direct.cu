// dt_direct.cu — persistent direct exchange plans (SURVEY §8(f) f1 across GPUs).
//
// The paper's GPU<->GPU path packs into a staging buffer, moves it, and unpacks
// on the receiver, pipelined so that the cost approaches "the cost of the data
// transfer plus the cost of the most expensive operation (pack or unpack) on a
// single fragment" ([L18:c4932 §4.1]).  With NVLink peer memory the sender can
// address the receiver's HBM directly, so the three stages collapse into one:
// the sending kernel walks its own layout and the RECEIVER's layout together
// (the fused datatype -> datatype copy of dt_copy) and stores every stream byte
// at its final address in peer memory.  No ring, no packed intermediate, no
// receiver-side unpack: each byte is read once from local HBM and written once
// into remote HBM.  The receiver's flattened type is shipped once at connect
// (dt_type_serialize) and committed on the sender's device.
//
// A plan is a fixed set of sends and receives (MPI persistent requests; the C4
// halo's 6 + 6 faces).  dt_xplan_start launches ONE cooperative kernel per rank:
//   CTA 0     posts every receive ("ready" = seq, release.sys store into the
//             source's flag page), then waits until every receive is "done";
//   CTAs 1..  belong to the sends: wait for the receiver's "ready", copy their
//             share of the message into the peer layout, fence.sys, count; the
//             last CTA of a send publishes "done" = seq into the receiver's page.
// Sequence numbers make the flags reusable without resets.
#include <cuda_runtime.h>
#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "dt_device.cuh"
#include "dt_internal.h"

namespace dt {

constexpr int kMaxDOps = 16;
constexpr int kDirThreads = 256;

struct DOp {
  KP S, R;               // source layout (local) and destination layout (peer memory)
  int32_t kind, g;       // 1 dual block walk, 2 dual word tables, 4 smem-staged; word size
  int32_t cta0, ncta;
  int64_t n;             // bytes of the message
  int64_t per;           // kind 1: stream bytes per warp
  int64_t ntiles;        // kind 4: 16 KiB tiles
  const uint64_t* ready; // local flag, written by the receiver: buffer posted for seq
  uint64_t* done;        // receiver's flag (peer memory): all bytes of seq landed
  uint32_t* cnt;         // local: CTAs of this send finished (cumulative over starts)
};

struct DArgs {
  int32_t nops, nrecv, wt_off, pad;
  uint64_t seq;
  int64_t timeout_ns;
  int32_t* err;
  uint64_t* post[kMaxDOps];           // per receive: "ready" flag in the source's page
  const uint64_t* arrived[kMaxDOps];  // per receive: local "done" flag
  DOp ops[kMaxDOps];
};

template <int G>
__device__ __forceinline__ void direct_words(const DOp& X, const int32_t* wts, const int32_t* wtr, int j) {
  dual_words<G, 4>(X.S, wts, X.R, wtr, 0, X.n, (int64_t)j * blockDim.x + threadIdx.x,
                   (int64_t)X.ncta * blockDim.x);
}

__global__ void __launch_bounds__(kDirThreads) k_direct(const __grid_constant__ DArgs A) {
  extern __shared__ __align__(128) uint8_t dsm[];
  __shared__ int s_stop;
  const uint64_t seq = A.seq;
  if (blockIdx.x == 0) {  // control CTA: post the receives, then wait for them
    for (int i = threadIdx.x; i < A.nrecv; i += blockDim.x) st_release_sys(A.post[i], seq);
    for (int i = threadIdx.x; i < A.nrecv; i += blockDim.x) {
      uint64_t v;
      spin(A.arrived[i], [seq](uint64_t x) { return x >= seq; }, A.timeout_ns, A.err, &v);
    }
    return;
  }
  int op = 0;
  for (int i = 0; i < A.nops; i++)
    if ((int)blockIdx.x >= A.ops[i].cta0 && (int)blockIdx.x < A.ops[i].cta0 + A.ops[i].ncta) op = i;
  const DOp& X = A.ops[op];
  const int j = (int)blockIdx.x - X.cta0;
  int32_t* wts = reinterpret_cast<int32_t*>(dsm + A.wt_off);
  int32_t* wtr = wts + X.S.nwords;
  if (X.kind != 1) {
    for (int i = threadIdx.x; i < X.S.nwords; i += blockDim.x) wts[i] = X.S.wtab[i];
    for (int i = threadIdx.x; i < X.R.nwords; i += blockDim.x) wtr[i] = X.R.wtab[i];
  }
  if (threadIdx.x == 0) {
    uint64_t v;
    s_stop = spin(X.ready, [seq](uint64_t x) { return x >= seq; }, A.timeout_ns, A.err, &v) ? 0 : 1;
  }
  __syncthreads();
  if (s_stop) return;
  if (X.kind == 1) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = (int64_t)j * (blockDim.x >> 5) + (threadIdx.x >> 5);
    const int64_t p = gw * X.per;
    if (p < X.n) dual_walk(X.S, X.R, p, min(p + X.per, X.n), lane);
  } else if (X.kind == 2) {
    switch (X.g) {
      case 1: direct_words<1>(X, wts, wtr, j); break;
      case 2: direct_words<2>(X, wts, wtr, j); break;
      case 4: direct_words<4>(X, wts, wtr, j); break;
      case 8: direct_words<8>(X, wts, wtr, j); break;
      default: direct_words<16>(X, wts, wtr, j); break;
    }
  } else {
    const int64_t t0 = X.ntiles * j / X.ncta, t1 = X.ntiles * (j + 1) / X.ncta;
    const int64_t lo = t0 * kStageTile, hi = min(t1 * (int64_t)kStageTile, X.n);
    if (lo < hi) {
      if (X.g == 4) stage_copy<4, kStageBufs>(X.S, wts, X.R, wtr, lo, hi, dsm);
      else if (X.g == 8) stage_copy<8, kStageBufs>(X.S, wts, X.R, wtr, lo, hi, dsm);
      else stage_copy<16, kStageBufs>(X.S, wts, X.R, wtr, lo, hi, dsm);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();  // this CTA's peer stores are visible system-wide before it counts
    const uint32_t old = atomicAdd(X.cnt, 1u);
    if (old + 1 == (uint32_t)(seq * (uint64_t)X.ncta)) {
      __threadfence_system();
      st_release_sys(X.done, seq);
    }
  }
}

// ------------------------------------------------------------------ host side
static dt_status cfail(cudaError_t e, const char* what) {
  set_error("%s: %s", what, cudaGetErrorString(e));
  return DT_ERR_CUDA;
}
#define CUD(call)                                    \
  do {                                               \
    cudaError_t _e = (call);                         \
    if (_e != cudaSuccess) return cfail(_e, #call);  \
  } while (0)

// process-wide cache of opened IPC handles (a handle may be opened once per process)
static std::mutex g_ipc_mu;
static std::map<std::string, std::pair<void*, int>> g_ipc;
static std::string ipc_key(const cudaIpcMemHandle_t& h) { return std::string(h.reserved, sizeof(h.reserved)); }
static dt_status ipc_map(const cudaIpcMemHandle_t& h, void** out) {
  std::lock_guard<std::mutex> g(g_ipc_mu);
  auto k = ipc_key(h);
  auto it = g_ipc.find(k);
  if (it != g_ipc.end()) {
    it->second.second++;
    *out = it->second.first;
    return DT_OK;
  }
  void* p = nullptr;
  CUD(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  g_ipc[k] = {p, 1};
  *out = p;
  return DT_OK;
}
static void ipc_unmap(const std::string& k) {
  std::lock_guard<std::mutex> g(g_ipc_mu);
  auto it = g_ipc.find(k);
  if (it == g_ipc.end()) return;
  if (--it->second.second == 0) {
    cudaIpcCloseMemHandle(it->second.first);
    g_ipc.erase(it);
  }
}

// base and size of the allocation holding p (driver cuMemGetAddressRange)
typedef int (*PfnGetRange)(unsigned long long*, size_t*, unsigned long long);
static dt_status alloc_base(const void* p, uint8_t** base) {
  static PfnGetRange fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    CUD(cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q));
    if (!f || q != cudaDriverEntryPointSuccess) {
      set_error("cuMemGetAddressRange unavailable");
      return DT_ERR_CUDA;
    }
    fn = (PfnGetRange)f;
  }
  unsigned long long b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, (unsigned long long)(uintptr_t)p) != 0) {
    set_error("cuMemGetAddressRange failed (not device memory?)");
    return DT_ERR_ARG;
  }
  *base = (uint8_t*)(uintptr_t)b;
  return DT_OK;
}

struct BlobHdr {
  uint32_t magic;
  int32_t rank;
  int64_t pid;
  int32_t device, nsend, nrecv, pad;
  uint64_t flags_ptr;
  cudaIpcMemHandle_t flags_h;
};
struct BlobSend {
  int32_t dest, tag, ready_idx, pad;
};
struct BlobRecv {
  int32_t source, tag, done_idx, pad;
  int64_t count, capacity, offset, type_len;
  uint64_t base_ptr;
  cudaIpcMemHandle_t h;
};
static const uint32_t kPlanMagic = 0xD1EC7A11u;

}  // namespace dt

using namespace dt;

struct dt_xplan_s {
  int rank = 0, nranks = 1, device = 0;
  std::vector<dt_xop> sends, recvs;
  uint64_t* flags = nullptr;  // [kMaxDOps ready][kMaxDOps done][kMaxDOps counters]
  int32_t* err = nullptr;
  uint64_t seq = 0;
  bool connected = false;
  DArgs A;
  unsigned grid = 0;
  size_t smem = 0;
  std::vector<dt_t> rtypes;          // receivers' types rebuilt on this device (owned)
  std::vector<std::string> mapped;   // IPC handles this plan opened
};

extern "C" {

dt_status dt_xplan_create(dt_comm_t c, int nsend, const dt_xop* sends, int nrecv, const dt_xop* recvs,
                          dt_xplan_t* out) {
  if (!c || !out || nsend < 0 || nrecv < 0 || nsend > kMaxDOps || nrecv > kMaxDOps || (nsend && !sends) ||
      (nrecv && !recvs)) {
    set_error("dt_xplan_create: bad argument (at most %d sends and %d receives)", kMaxDOps, kMaxDOps);
    return DT_ERR_ARG;
  }
  auto* p = new dt_xplan_s;
  comm_info(c, &p->rank, &p->nranks, &p->device);
  p->sends.assign(sends, sends + nsend);
  p->recvs.assign(recvs, recvs + nrecv);
  auto bad = [&](const char* m) {
    delete p;
    set_error("dt_xplan_create: %s", m);
    return DT_ERR_ARG;
  };
  for (auto& o : p->sends) {
    if (!o.type || o.count < 0 || o.peer < 0 || o.peer >= p->nranks) return bad("bad send");
    if (!o.type->committed) {
      delete p;
      set_error("dt_xplan_create: send type not committed");
      return DT_ERR_NOT_COMMITTED;
    }
  }
  for (auto& o : p->recvs) {
    if (!o.type || o.count < 0 || o.peer < 0 || o.peer >= p->nranks) return bad("bad receive");
    if (!o.type->committed) {
      delete p;
      set_error("dt_xplan_create: receive type not committed");
      return DT_ERR_NOT_COMMITTED;
    }
    if (nonoverlap_cached(o.type, o.count) != 1) {
      delete p;
      set_error("dt_xplan_create: receive typemap entries overlap");
      return DT_ERR_OVERLAP;
    }
  }
  for (size_t a = 0; a < p->sends.size(); a++)
    for (size_t b = a + 1; b < p->sends.size(); b++)
      if (p->sends[a].peer == p->sends[b].peer && p->sends[a].tag == p->sends[b].tag) return bad("duplicate send tag");
  for (size_t a = 0; a < p->recvs.size(); a++)
    for (size_t b = a + 1; b < p->recvs.size(); b++)
      if (p->recvs[a].peer == p->recvs[b].peer && p->recvs[a].tag == p->recvs[b].tag)
        return bad("duplicate receive tag");
  cudaError_t e = cudaSetDevice(p->device);
  if (e == cudaSuccess) e = cudaMalloc(&p->flags, 3 * kMaxDOps * sizeof(uint64_t));
  if (e == cudaSuccess) e = cudaMemset(p->flags, 0, 3 * kMaxDOps * sizeof(uint64_t));
  if (e == cudaSuccess) e = cudaMalloc(&p->err, sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMemset(p->err, 0, sizeof(int32_t));
  if (e != cudaSuccess) {
    cudaFree(p->flags);
    cudaFree(p->err);
    delete p;
    return cfail(e, "dt_xplan_create alloc");
  }
  *out = p;
  return DT_OK;
}

dt_status dt_xplan_local_blob(dt_xplan_t p, void* out, size_t* nbytes) {
  if (!p || !nbytes) {
    set_error("dt_xplan_local_blob: NULL");
    return DT_ERR_ARG;
  }
  std::vector<uint8_t> b(sizeof(BlobHdr));
  BlobHdr h;
  std::memset(&h, 0, sizeof(h));
  h.magic = kPlanMagic;
  h.rank = p->rank;
  h.pid = (int64_t)getpid();
  h.device = p->device;
  h.nsend = (int32_t)p->sends.size();
  h.nrecv = (int32_t)p->recvs.size();
  h.flags_ptr = (uint64_t)(uintptr_t)p->flags;
  CUD(cudaSetDevice(p->device));
  CUD(cudaIpcGetMemHandle(&h.flags_h, p->flags));
  std::memcpy(b.data(), &h, sizeof(h));
  for (size_t i = 0; i < p->sends.size(); i++) {
    BlobSend s{p->sends[i].peer, p->sends[i].tag, (int32_t)i, 0};
    const size_t o = b.size();
    b.resize(o + sizeof(s));
    std::memcpy(b.data() + o, &s, sizeof(s));
  }
  for (size_t j = 0; j < p->recvs.size(); j++) {
    const dt_xop& r = p->recvs[j];
    BlobRecv x;
    std::memset(&x, 0, sizeof(x));
    x.source = r.peer;
    x.tag = r.tag;
    x.done_idx = kMaxDOps + (int32_t)j;
    x.count = r.count;
    x.capacity = r.count * r.type->size;
    uint8_t* base = nullptr;
    dt_status st = alloc_base((uint8_t*)r.buf + r.type->true_lb, &base);
    if (st != DT_OK) return st;
    x.base_ptr = (uint64_t)(uintptr_t)base;
    x.offset = (int64_t)((uint8_t*)r.buf - base);
    CUD(cudaIpcGetMemHandle(&x.h, base));
    size_t tl = 0;
    st = dt_type_serialize(r.type, nullptr, &tl);
    if (st != DT_OK) return st;
    x.type_len = (int64_t)tl;
    const size_t o = b.size();
    b.resize(o + sizeof(x) + tl);
    std::memcpy(b.data() + o, &x, sizeof(x));
    st = dt_type_serialize(r.type, b.data() + o + sizeof(x), &tl);
    if (st != DT_OK) return st;
  }
  if (!out) {
    *nbytes = b.size();
    return DT_OK;
  }
  if (*nbytes < b.size()) {
    set_error("dt_xplan_local_blob: buffer too small");
    return DT_ERR_ARG;
  }
  std::memcpy(out, b.data(), b.size());
  *nbytes = b.size();
  return DT_OK;
}

dt_status dt_xplan_connect(dt_xplan_t p, const void* blobs, const size_t* sizes) {
  if (!p || !blobs || !sizes) {
    set_error("dt_xplan_connect: NULL");
    return DT_ERR_ARG;
  }
  if (p->connected) {
    set_error("dt_xplan_connect: already connected");
    return DT_ERR_ARG;
  }
  CUD(cudaSetDevice(p->device));
  // parse every rank's blob
  struct Parsed {
    BlobHdr h;
    std::vector<BlobSend> s;
    std::vector<BlobRecv> r;
    std::vector<const uint8_t*> tbytes;
  };
  std::vector<Parsed> P((size_t)p->nranks);
  const uint8_t* cur = (const uint8_t*)blobs;
  for (int r = 0; r < p->nranks; r++) {
    const uint8_t* q = cur;
    const uint8_t* end = cur + sizes[r];
    cur = end;
    if (sizes[r] < sizeof(BlobHdr)) {
      set_error("dt_xplan_connect: short blob from rank %d", r);
      return DT_ERR_ARG;
    }
    std::memcpy(&P[r].h, q, sizeof(BlobHdr));
    q += sizeof(BlobHdr);
    if (P[r].h.magic != kPlanMagic || P[r].h.rank != r) {
      set_error("dt_xplan_connect: malformed blob of rank %d", r);
      return DT_ERR_ARG;
    }
    for (int i = 0; i < P[r].h.nsend; i++) {
      BlobSend s;
      std::memcpy(&s, q, sizeof(s));
      q += sizeof(s);
      P[r].s.push_back(s);
    }
    for (int i = 0; i < P[r].h.nrecv; i++) {
      BlobRecv x;
      if (q + sizeof(x) > end) {
        set_error("dt_xplan_connect: truncated blob of rank %d", r);
        return DT_ERR_ARG;
      }
      std::memcpy(&x, q, sizeof(x));
      q += sizeof(x);
      P[r].r.push_back(x);
      P[r].tbytes.push_back(q);
      q += x.type_len;
    }
  }
  const int64_t mypid = (int64_t)getpid();
  auto remote = [&](int r, uint64_t ptr, const cudaIpcMemHandle_t& h, uint8_t** out) -> dt_status {
    if (r == p->rank || P[r].h.pid == mypid) {  // same process: plain pointer (peer access if another GPU)
      if (P[r].h.device != p->device) {
        cudaError_t e = cudaDeviceEnablePeerAccess(P[r].h.device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return cfail(e, "cudaDeviceEnablePeerAccess");
        cudaGetLastError();
      }
      *out = (uint8_t*)(uintptr_t)ptr;
      return DT_OK;
    }
    void* m = nullptr;
    dt_status st = ipc_map(h, &m);
    if (st != DT_OK) return st;
    p->mapped.push_back(ipc_key(h));
    *out = (uint8_t*)m;
    return DT_OK;
  };
  DArgs& A = p->A;
  std::memset(&A, 0, sizeof(A));
  A.err = p->err;
  const char* to = getenv("DT_TIMEOUT_MS");
  A.timeout_ns = (int64_t)(to ? atoll(to) : 30000) * 1000000ll;
  // receives: where to post "ready" (the matching send's slot in the source's page)
  A.nrecv = (int32_t)p->recvs.size();
  for (size_t j = 0; j < p->recvs.size(); j++) {
    const dt_xop& r = p->recvs[j];
    const Parsed& src = P[r.peer];
    int idx = -1;
    for (auto& s : src.s)
      if (s.dest == p->rank && s.tag == r.tag) idx = s.ready_idx;
    if (idx < 0) {
      set_error("dt_xplan_connect: rank %d has no send (dest %d, tag %d) for this receive", r.peer, p->rank, r.tag);
      return DT_ERR_ARG;
    }
    uint8_t* fl = nullptr;
    dt_status st = remote(r.peer, src.h.flags_ptr, src.h.flags_h, &fl);
    if (st != DT_OK) return st;
    A.post[j] = reinterpret_cast<uint64_t*>(fl) + idx;
    A.arrived[j] = p->flags + kMaxDOps + j;
  }
  // sends: the receiver's layout in its memory, its type rebuilt here
  A.nops = (int32_t)p->sends.size();
  int64_t total = 0;
  bool any_stage = false;
  size_t wt_bytes = 0;
  for (size_t i = 0; i < p->sends.size(); i++) {
    const dt_xop& s = p->sends[i];
    const Parsed& dst = P[s.peer];
    int k = -1;
    for (size_t q = 0; q < dst.r.size(); q++)
      if (dst.r[q].source == p->rank && dst.r[q].tag == s.tag) k = (int)q;
    if (k < 0) {
      set_error("dt_xplan_connect: rank %d has no receive (source %d, tag %d) for this send", s.peer, p->rank, s.tag);
      return DT_ERR_ARG;
    }
    const BlobRecv& R = dst.r[k];
    const int64_t n = s.count * s.type->size;
    if (n > R.capacity) {
      set_error("dt_xplan_connect: send of %lld bytes to rank %d tag %d exceeds the %lld-byte receive", (long long)n,
                s.peer, s.tag, (long long)R.capacity);
      return DT_ERR_TRUNCATE;
    }
    dt_t rt = nullptr;
    dt_status st = dt_type_deserialize(dst.tbytes[k], (size_t)R.type_len, &rt);
    if (st != DT_OK) return st;
    p->rtypes.push_back(rt);
    st = dt_commit(rt);
    if (st != DT_OK) return st;
    uint8_t* rbase = nullptr;
    st = remote(s.peer, R.base_ptr, R.h, &rbase);
    if (st != DT_OK) return st;
    uint8_t* fl = nullptr;
    st = remote(s.peer, dst.h.flags_ptr, dst.h.flags_h, &fl);
    if (st != DT_OK) return st;
    DOp& X = A.ops[i];
    X.n = n;
    X.ready = p->flags + i;
    X.done = reinterpret_cast<uint64_t*>(fl) + R.done_idx;
    X.cnt = reinterpret_cast<uint32_t*>(p->flags + 2 * kMaxDOps + i);
    X.kind = 1;
    X.g = 1;
    if (n > 0) {
      int kind = 1;
      int64_t g = 1;
      st = dual_params(s.type, s.count, s.buf, rt, R.count, rbase + R.offset, n, X.S, X.R, &kind, &g);
      if (st != DT_OK) return st;
      X.kind = kind;
      X.g = (int32_t)g;
      if (kind != 1) wt_bytes = std::max(wt_bytes, sizeof(int32_t) * (size_t)(X.S.nwords + X.R.nwords));
      any_stage = any_stage || kind == 4;
    }
    total += n;
  }
  // launch shape: CTA 0 controls, the sends share the co-resident rest by bytes x a
  // per-family cost (G-byte word gathers/scatters move bytes ~16/G times slower per CTA
  // than long runs: the C4 x faces next to the y/z faces)
  A.wt_off = any_stage ? kStageBufs * kStageTile : 0;
  p->smem = (size_t)A.wt_off + wt_bytes;
  CUD(cudaFuncSetAttribute(k_direct, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)std::max<size_t>(p->smem, 1)));
  int occ = 0, sms = 0;
  CUD(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct, kDirThreads, p->smem));
  CUD(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p->device));
  const char* mc = getenv("DT_DIRECT_CTAS");  // f3: cap the CTAs the sends may use
  int budget = occ * sms - 1;
  if (mc && atoi(mc) > 0) budget = std::min(budget, atoi(mc));
  if (budget < A.nops) {
    set_error("dt_xplan_connect: %d sends need more co-resident CTAs than the device offers", A.nops);
    return DT_ERR_UNSUPPORTED;
  }
  auto cost = [](const DOp& X) { return (double)X.n * ((X.kind == 2 || X.kind == 4) ? 16.0 / X.g : 1.0); };
  double ctot = 0;
  for (int i = 0; i < A.nops; i++) ctot += cost(A.ops[i]);
  int next = 1;
  int left = budget;
  for (int i = 0; i < A.nops; i++) {
    DOp& X = A.ops[i];
    const int rest = A.nops - i - 1;  // keep one CTA for every later send
    int want = ctot > 0 ? (int)((double)budget * cost(X) / ctot) : 1;
    want = std::max(1, std::min(want, (int)std::max<int64_t>(1, X.n / 16384)));
    want = std::min(want, left - rest);
    X.cta0 = next;
    X.ncta = want;
    next += want;
    left -= want;
    const int64_t nw = (int64_t)X.ncta * (kDirThreads / 32);
    X.per = std::max<int64_t>(512, ((X.n + nw - 1) / nw + 511) & ~int64_t(511));
    X.ntiles = (X.n + kStageTile - 1) / kStageTile;
  }
  p->grid = (unsigned)next;
  p->connected = true;
  return DT_OK;
}

dt_status dt_xplan_start(dt_xplan_t p, void* stream) {
  if (!p || !p->connected) {
    set_error("dt_xplan_start: plan not connected");
    return DT_ERR_ARG;
  }
  CUD(cudaSetDevice(p->device));
  p->A.seq = ++p->seq;
  void* args[] = {(void*)&p->A};
  CUD(cudaLaunchCooperativeKernel((const void*)k_direct, dim3(p->grid), dim3(kDirThreads), args, p->smem,
                                  (cudaStream_t)stream));
  return DT_OK;
}

dt_status dt_xplan_check(dt_xplan_t p) {
  if (!p) {
    set_error("dt_xplan_check: NULL");
    return DT_ERR_ARG;
  }
  int32_t e = 0;
  CUD(cudaSetDevice(p->device));
  CUD(cudaMemcpy(&e, p->err, sizeof(e), cudaMemcpyDeviceToHost));
  if (e) {
    set_error("dt_xplan: a peer flag wait timed out (DT_TIMEOUT_MS)");
    return DT_ERR_TIMEOUT;
  }
  return DT_OK;
}

dt_status dt_xplan_free(dt_xplan_t* pp) {
  if (!pp) {
    set_error("dt_xplan_free: NULL");
    return DT_ERR_ARG;
  }
  dt_xplan_s* p = *pp;
  if (p) {
    cudaSetDevice(p->device);
    cudaDeviceSynchronize();
    for (auto& k : p->mapped) ipc_unmap(k);
    for (auto& t : p->rtypes) dt_free(&t);
    cudaFree(p->flags);
    cudaFree(p->err);
    delete p;
  }
  *pp = nullptr;
  return DT_OK;
}

}  // extern "C"
