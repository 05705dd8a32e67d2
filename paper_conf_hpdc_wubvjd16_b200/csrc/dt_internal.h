// dt_internal.h — private structures of libdt (host type system, GPU descriptor,
// kernel parameters).  Not part of the C-ABI (include/dt.h is).
#pragma once
#include <cstdint>
#include <cstdlib>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/dt.h"

namespace dt {

constexpr int kMaxLevels = 8;          // levels a kernel walks (incl. the instance level)
constexpr int64_t kMaxFlatBlocks = int64_t(1) << 28;  // cap on an expanded block list
constexpr int64_t kMaxWordTable = 12288;              // word-table kernel: entries in smem

void set_error(const char* fmt, ...);

// Smallest word size G the smem/TMA staged family takes (cp.async gathers, persistent
// element iterators); below it the register word-table family.  4 since round 2 (C4
// x-face 1 MiB: staged pack/unpack 15.4 / 13.3 us vs 17.4 / 20.5 on 148 SMs, 21.5 vs
// 44 us on 16 SMs); DT_STAGE_G=8 restores the round-1 rule.
inline int64_t stage_min_g() {
  static const int64_t g = [] {
    const char* e = std::getenv("DT_STAGE_G");
    return e && std::atoll(e) > 0 ? (int64_t)std::atoll(e) : (int64_t)4;
  }();
  return g;
}

// One level of the element iteration space above the block template.
// Element index decomposes mixed-radix over the levels, the LAST level fastest
// (typemap order: outer constructor loops are slow).  A regular level
// contributes idx*stride bytes, a list level contributes table[idx] bytes.
struct Level {
  int64_t cnt = 1;
  int64_t stride = 0;
  std::shared_ptr<std::vector<int64_t>> table;  // non-null => list level
  bool is_list() const { return table != nullptr; }
  int64_t contrib(int64_t i) const { return table ? (*table)[i] : i * stride; }
};

// Flattened form of one type instance: for each element e (in typemap order)
// the template blocks (bd[i] + disp(e), bl[i]) in order.  This is the B200
// re-encoding of the paper's DEV list ([L16:c5201 §3.2]): regular nests stay
// implicit (the paper's vector kernel, [L16:c2243 §3.1]) and only irregular
// parts are listed.
struct Form {
  std::vector<Level> lv;           // outermost first
  std::vector<int64_t> bd, bl;     // template blocks (bytes), typemap order
  // per-call planning must stay O(levels): O(n) facts are computed once and cached
  mutable int64_t gran_cache = -1, tsize_cache = -1, lvl_gran_cache = -1;
  mutable int fits32_cache = -1;
  mutable int span_local_cache = -1;  // block-span kernel: are 32-block windows locally dense?
  mutable int sdesc_ok_cache = -1;    // do the blocks fit the compact span descriptors?
  mutable int64_t span_lo = 0, span_hi = -1;  // cached min bd / max bd+bl (span_hi < span_lo: not computed)
  // f2 GPU-side flattening: the merged block list was built on the device and the host
  // arrays bd/bl stay empty until a host consumer asks for them (materialize_host);
  // nb_dev blocks, the first block (bd0_dev, bl0_dev), and whether the blocks are sorted
  // and disjoint (mono_dev, the unpack legality fact) come from the device pass
  int64_t nb_dev = -1, bd0_dev = 0, bl0_dev = 0;
  int mono_dev = -1;
  bool host_missing() const { return nb_dev >= 0; }  // (materialize_host resets nb_dev to -1)
  int64_t nblocks() const { return host_missing() ? nb_dev : (int64_t)bl.size(); }
  int64_t first_bd() const { return host_missing() ? bd0_dev : bd.empty() ? 0 : bd[0]; }
  int64_t first_bl() const { return host_missing() ? bl0_dev : bl.empty() ? 0 : bl[0]; }
  void span(int64_t* lo, int64_t* hi) const {
    if (span_hi < span_lo) {
      int64_t a = INT64_MAX, b = INT64_MIN;
      for (size_t i = 0; i < bd.size(); i++) {
        a = bd[i] < a ? bd[i] : a;
        b = bd[i] + bl[i] > b ? bd[i] + bl[i] : b;
      }
      span_lo = a;
      span_hi = b;
    }
    *lo = span_lo;
    *hi = span_hi;
  }
  int64_t tsize() const {
    if (tsize_cache < 0) { int64_t s = 0; for (auto x : bl) s += x; tsize_cache = s; }
    return tsize_cache;
  }
  mutable std::vector<int64_t> hoff_cache;  // host exclusive prefix of bl (launch planning)
  void invalidate() const {
    if (host_missing()) return;  // (device facts stay: the device form is never edited)
    gran_cache = tsize_cache = lvl_gran_cache = -1;
    fits32_cache = -1;
    span_local_cache = -1;
    sdesc_ok_cache = -1;
    span_lo = 0;
    span_hi = -1;
    hoff_cache.clear();
  }
  const std::vector<int64_t>& hoff() const {
    if (hoff_cache.size() != bl.size()) {
      hoff_cache.resize(bl.size());
      int64_t s = 0;
      for (size_t i = 0; i < bl.size(); i++) { hoff_cache[i] = s; s += bl[i]; }
    }
    return hoff_cache;
  }
  int64_t nelem() const { int64_t n = 1; for (auto& l : lv) n *= l.cnt; return n; }
  bool empty() const { return nblocks() == 0; }
};

void normalize(Form& f);
struct DeviceDesc;
// f2: download a device-flattened form's block list into its host arrays (no-op when
// present); dd: a descriptor holding it
dt_status materialize_host(const Form& f, const DeviceDesc& dd);
// Expand into merged blocks (typemap order).  Returns false if > cap.
bool expand(const Form& f, std::vector<int64_t>& d, std::vector<int64_t>& l, int64_t cap);
int64_t form_granularity(const Form& f);
// largest power of two <= 16 dividing every level stride / list entry (element bases)
int64_t level_granularity(const Form& f);

// Per-device copy of the descriptor.
struct DeviceDesc {
  int device = -1;
  int64_t* bd = nullptr;    // template disps
  int64_t* bl = nullptr;    // template lens
  int64_t* boff = nullptr;  // exclusive prefix of bl (device scan)
  std::vector<int64_t*> tables;  // per level (nullptr for regular levels)
  // word tables for the short kernel, keyed by granularity (1,2,4,8,16)
  int32_t* wtab[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};
  // compact block descriptors of the block-span kernel (built on first use; state
  // -1 unknown, 0 not representable, 1 built)
  uint64_t* sdesc = nullptr;
  int64_t* wbase = nullptr;
  int sdesc_state = -1;
  // cached cost-balanced warp plans of the long-run kernel, keyed by the launch shape
  struct PlanSlot {
    int64_t count = -1, pos = 0, len = 0, nw = 0, alpha = 0, tsize = 0, gran = 1;
    void* d = nullptr;
    void* made_on = nullptr;  // stream the k_plan that filled `d` was enqueued on
    void* ready = nullptr;    // cudaEvent_t recorded after that k_plan (cross-stream reuse waits on it)
  };
  std::vector<PlanSlot> plans;
  size_t plan_next = 0;
};

enum Kind { K_BASIC, K_CONTIG, K_HVECTOR, K_HINDEXED, K_STRUCT, K_SUBARRAY, K_RESIZED, K_FLAT };
// K_FLAT: a type rebuilt from its serialized flattened form (dt_type_deserialize);
// its Form is stored at creation and it has no constructor tree.

}  // namespace dt

struct dt_type_s {
  int refcnt = 1;
  bool predefined = false;
  dt::Kind kind = dt::K_BASIC;
  int basic = 0;
  int64_t count = 0, blocklen = 0, stride = 0;           // stride in bytes
  std::vector<int64_t> bls, dps;                          // bytes (struct; hindexed: bls only when not uniform)
  std::shared_ptr<std::vector<int64_t>> hdps;             // hindexed displacements (bytes), shared with the form
  std::vector<dt_type_s*> types;                          // struct components
  int ndims = 0, order = 0;
  std::vector<int64_t> sizes, subsizes, starts;
  dt_type_s* old = nullptr;
  // bounds
  int64_t size = 0, lb = 0, ub = 0, true_lb = 0, true_ub = 0, align = 1;
  bool has_lb = false, has_ub = false;
  // commit state
  std::mutex mu;
  bool committed = false;
  std::unique_ptr<dt::Form> form;        // host form (built lazily)
  std::vector<dt::DeviceDesc> devs;      // per device uploads
  // f2: commit deferred the flattening of a huge block list to the first whole-stream
  // pack, which flattens, uploads and packs it in a pipeline
  bool lazy_pipe = false;
  // overlap cache (unpack legality) for the last count checked
  int64_t ovl_count = -1;
  int ovl_result = 0;
  int64_t extent() const { return ub - lb; }
};

namespace dt {
// kernels.cu
struct KLevels {
  int n = 0;
  int64_t cnt[kMaxLevels];
  int64_t stride[kMaxLevels];
  const int64_t* table[kMaxLevels];
};
dt_status upload_desc(dt_type_s* t, const Form& f, DeviceDesc& dd);
void free_desc(DeviceDesc& dd);
dt_status launch_pack_unpack(bool unpack, dt_type_s* t, const Form& f, DeviceDesc& dd, int64_t count,
                             const void* nc, void* c, int64_t pos, int64_t len, void* stream);
int plan_kernel(const Form& f, const KLevels& L, uint64_t nc_addr, uint64_t c_addr, int64_t pos, int64_t len,
                int64_t* gran);
void build_levels(const Form& f, const DeviceDesc* dd, dt_type_s* t, int64_t count, KLevels& L);
// Effective template of one launch: a single-block template whose innermost regular
// level continues the run (count instances of a contiguous type, a vector of
// adjacent blocks) becomes one longer run when that makes it a long-run copy.
struct Eff {
  KLevels L;
  int64_t tsize, nblocks, bd0, bl0;
  bool merged;
};
Eff effective(const Form& f, const DeviceDesc* dd, dt_type_s* t, int64_t count);
// f2 pipelined first use (dt_types.cpp): is t an hindexed list of a contiguous element
// with per-entry lengths (the block list flattens entry by entry)?  d0/l0: the element's
// run.  install_form: adopt a form built outside build_form.  huge_reserve: reserve a
// large vector on transparent huge pages.
bool pipe_list(dt_type_s* t, int64_t* d0, int64_t* l0);
void install_form(dt_type_s* t, Form&& f);
void huge_reserve(std::vector<int64_t>& v, size_t n);
dt_status ensure_committed_on_device(dt_type_s* t, DeviceDesc** out);
const Form& get_form(dt_type_s* t);
// xfer.cu: identity of a communicator (direct exchange plans live beside it)
void comm_info(dt_comm_t c, int* rank, int* nranks, int* device);
dt_status ensure_wtab_pub(const Form& f, DeviceDesc& dd, int64_t g, const int32_t** out);
// compact (8-byte) block descriptors for the block-span kernel, or nullptrs when a
// block does not fit (|disp - group base| >= 2^31 or len >= 2^32)
dt_status ensure_sdesc(const Form& f, DeviceDesc& dd, const uint64_t** sdesc, const int64_t** wbase);
}  // namespace dt
