// dt_types.cpp — host type system of libdt: MPI constructors, bounds, and the
// commit-time flattening into a GPU descriptor (Form = strided/list levels over
// a merged (disp,len) block template).
//
// Paper: the host "simulates the pack" and produces relative displacements that
// depend only on the layout, so they are cached ([L16:c1326 §3], [L16:c1579 §3]);
// DEVs = (packed disp, non-contig disp, blocklength) [L16:c5201 §3.2]; the vector
// specialisation needs no list at all [L16:c2243 §3.1].  Here regular nests
// (vector/hvector/subarray/contiguous) stay implicit as levels and only
// irregular displacements become lists, so the descriptor of a 1 GB message
// never becomes a 1 GB DEV array (SURVEY §7 hard part 3).
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <thread>

#include <sys/mman.h>

#include "dt_internal.h"

namespace dt {

static thread_local char g_err[512] = "";
void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

static const int64_t kBasicSize[8] = {1, 1, 1, 2, 4, 8, 4, 8};

// Reserve a large vector on transparent huge pages (first-use cost, f2): a 1 GB
// index list has ~2e7-3e7 entries, and faulting 240 MB in 4 KiB pages costs more
// than the flattening arithmetic itself.
void huge_reserve(std::vector<int64_t>& v, size_t n) {
  v.reserve(n);
  const size_t bytes = n * sizeof(int64_t), hp = size_t(2) << 20;
  if (bytes < 4 * hp) return;
  const uintptr_t a = ((uintptr_t)v.data() + hp - 1) & ~(uintptr_t)(hp - 1);
  const uintptr_t e = ((uintptr_t)v.data() + bytes) & ~(uintptr_t)(hp - 1);
  if (e > a) madvise((void*)a, e - a, MADV_HUGEPAGE);
}
// Host threads for O(n) passes over huge index lists (first-use cost, f2): fn(lo, hi,
// thread) over [0, n) split into equal ranges; serial below 1M entries.
template <typename F>
static int parallel_for(size_t n, F fn) {
  const size_t kMin = size_t(1) << 20;
  int nt = 1;
  if (n >= kMin) {
    const unsigned hw = std::thread::hardware_concurrency();
    nt = (int)std::max(1u, std::min(16u, hw ? hw : 1u));
    const char* e = getenv("DT_HOST_THREADS");
    if (e && atoi(e) > 0) nt = std::min(64, atoi(e));
  }
  if (nt == 1) {
    fn((size_t)0, n, 0);
    return 1;
  }
  std::vector<std::thread> th;
  for (int t = 1; t < nt; t++) th.emplace_back(fn, n * t / nt, n * (t + 1) / nt, t);
  fn((size_t)0, n / nt, 0);
  for (auto& x : th) x.join();
  return nt;
}
static void huge_assign(std::vector<int64_t>& v, const int64_t* p, size_t n) {
  huge_reserve(v, n);
  v.resize(n);
  int64_t* d = v.data();
  parallel_for(n, [=](size_t lo, size_t hi, int) { std::memcpy(d + lo, p + lo, (hi - lo) * sizeof(int64_t)); });
}

// ------------------------------------------------------------------ bounds
// Bounds of a constructed type from the range of shifts its copies of T take
// (MPI-3.1 §4.1.6; readings R-markers, R-eps in DESIGN.md).
struct Bounds {
  bool lbm = false, ubm = false, data = false;
  int64_t lbv = 0, ubv = 0, dlb = 0, dub = 0, tlb = 0, tub = 0, size = 0, align = 1;
  // copies of T with shifts in [smin, smax], ncopies of them
  void add(const dt_type_s* T, int64_t smin, int64_t smax, int64_t ncopies) {
    if (ncopies <= 0) return;
    if (T->has_lb) { lbv = lbm ? std::min(lbv, smin + T->lb) : smin + T->lb; lbm = true; }
    if (T->has_ub) { ubv = ubm ? std::max(ubv, smax + T->ub) : smax + T->ub; ubm = true; }
    if (T->size > 0) {
      if (!data) { dlb = smin + T->lb; dub = smax + T->ub; tlb = smin + T->true_lb; tub = smax + T->true_ub; }
      else {
        dlb = std::min(dlb, smin + T->lb); dub = std::max(dub, smax + T->ub);
        tlb = std::min(tlb, smin + T->true_lb); tub = std::max(tub, smax + T->true_ub);
      }
      data = true;
    }
    size += T->size * ncopies;
    align = std::max(align, T->align);
  }
  void finish(dt_type_s* t, bool is_struct) {
    t->size = size;
    t->align = align;
    t->has_lb = lbm;
    t->has_ub = ubm;
    t->lb = lbm ? lbv : (data ? dlb : 0);
    t->ub = ubm ? ubv : (data ? dub : 0);
    if (is_struct && !ubm && data) {
      int64_t e = t->ub - t->lb;
      int64_t r = ((e % align) + align) % align;
      if (r) t->ub += align - r;
    }
    t->true_lb = data ? tlb : 0;
    t->true_ub = data ? tub : 0;
  }
};

// range of i*a for i in [0, n)
static inline void lin_range(int64_t n, int64_t a, int64_t& lo, int64_t& hi) {
  int64_t last = (n - 1) * a;
  lo = std::min<int64_t>(0, last);
  hi = std::max<int64_t>(0, last);
}

}  // namespace dt

using namespace dt;

static dt_type_s g_basic[8];
static std::once_flag g_basic_once;
static void init_basics() {
  for (int k = 0; k < 8; k++) {
    dt_type_s& b = g_basic[k];
    b.predefined = true;
    b.kind = K_BASIC;
    b.basic = k;
    b.size = kBasicSize[k];
    b.lb = 0;
    b.ub = b.size;
    b.true_lb = 0;
    b.true_ub = b.size;
    b.align = b.size;
  }
}

static dt_type_s* retain(dt_type_s* t) {
  if (!t->predefined) t->refcnt++;
  return t;
}
static void release(dt_type_s* t) {
  if (!t || t->predefined) return;
  if (--t->refcnt > 0) return;
  if (t->old) release(t->old);
  for (auto* c : t->types) release(c);
  for (auto& dd : t->devs) free_desc(dd);
  delete t;
}

#define CHECK_ARG(cond, msg)                   \
  do {                                         \
    if (!(cond)) {                             \
      set_error("%s: %s", __func__, msg);      \
      return DT_ERR_ARG;                       \
    }                                          \
  } while (0)

extern "C" {

dt_t dt_basic_type(dt_basic k) {
  std::call_once(g_basic_once, init_basics);
  if ((int)k < 0 || (int)k > 7) {
    set_error("dt_basic_type: invalid kind %d", (int)k);
    return nullptr;
  }
  return &g_basic[(int)k];
}

dt_status dt_create_hvector(int64_t count, int64_t blocklen, int64_t stride, dt_t old, dt_t* out) {
  CHECK_ARG(old && out, "NULL argument");
  CHECK_ARG(count >= 0 && blocklen >= 0, "negative count/blocklen");
  auto* t = new dt_type_s;
  t->kind = K_HVECTOR;
  t->count = count;
  t->blocklen = blocklen;
  t->stride = stride;
  t->old = retain(old);
  Bounds b;
  if (count > 0 && blocklen > 0) {
    int64_t a0, a1, b0, b1;
    lin_range(count, stride, a0, a1);
    lin_range(blocklen, old->extent(), b0, b1);
    b.add(old, a0 + b0, a1 + b1, count * blocklen);
  }
  b.finish(t, false);
  *out = t;
  return DT_OK;
}

dt_status dt_create_contiguous(int64_t count, dt_t old, dt_t* out) {
  CHECK_ARG(old && out, "NULL argument");
  CHECK_ARG(count >= 0, "negative count");
  dt_status s = dt_create_hvector(count, 1, old->extent(), old, out);
  if (s == DT_OK) (*out)->kind = K_CONTIG;
  return s;
}

dt_status dt_create_vector(int64_t count, int64_t blocklen, int64_t stride, dt_t old, dt_t* out) {
  CHECK_ARG(old && out, "NULL argument");
  return dt_create_hvector(count, blocklen, stride * old->extent(), old, out);
}

}  // extern "C"

// hindexed with per-entry blocklens (bls) or one uniform blocklen (bls == nullptr)
static dt_status create_hindexed(int64_t count, const int64_t* bls, int64_t ubl, const int64_t* dps, dt_t old,
                                 dt_t* out) {
  CHECK_ARG(old && out, "NULL argument");
  CHECK_ARG(count >= 0, "negative count");
  CHECK_ARG(count == 0 || dps, "NULL arrays");
  if (!bls) CHECK_ARG(ubl >= 0, "negative blocklen");
  // every copy is of the same type `old`, so the bounds need only the range of the
  // shifts over all copies and their number: one pass over the arrays (which also
  // validates the block lengths), before anything is allocated
  const int64_t e = old->extent();
  struct Part {
    int64_t smin = INT64_MAX, smax = INT64_MIN, ncopies = 0;
    bool neg = false;
  };
  Part parts[64];
  const int nt = parallel_for((size_t)count, [&](size_t i0, size_t i1, int t) {
    Part q;
    for (size_t i = i0; i < i1; i++) {
      const int64_t n = bls ? bls[i] : ubl;
      q.neg |= n < 0;
      if (n <= 0) continue;
      const int64_t last = (n - 1) * e;
      const int64_t lo = dps[i] + (last < 0 ? last : 0), hi = dps[i] + (last > 0 ? last : 0);
      q.smin = lo < q.smin ? lo : q.smin;
      q.smax = hi > q.smax ? hi : q.smax;
      q.ncopies += n;
    }
    parts[t] = q;
  });
  int64_t smin = INT64_MAX, smax = INT64_MIN, ncopies = 0;
  bool neg = false;
  for (int t = 0; t < nt; t++) {
    smin = std::min(smin, parts[t].smin);
    smax = std::max(smax, parts[t].smax);
    ncopies += parts[t].ncopies;
    neg |= parts[t].neg;
  }
  CHECK_ARG(!neg, "negative blocklen");
  auto* t = new dt_type_s;
  t->kind = K_HINDEXED;
  t->count = count;
  // f2 (first-use cost): a uniform block length is kept as one number, and the
  // displacement list is held once and shared with the flattened form's list level
  // (a 1 GB index list has ~2e7 entries; every extra copy of it is page faults)
  if (bls) huge_assign(t->bls, bls, (size_t)count);
  t->blocklen = bls ? -1 : ubl;
  t->hdps = std::make_shared<std::vector<int64_t>>();
  huge_assign(*t->hdps, dps, (size_t)count);
  t->old = retain(old);
  Bounds b;
  if (ncopies > 0) b.add(old, smin, smax, ncopies);
  b.finish(t, false);
  *out = t;
  return DT_OK;
}

extern "C" {

dt_status dt_create_hindexed(int64_t count, const int64_t* bls, const int64_t* dps, dt_t old, dt_t* out) {
  CHECK_ARG(count == 0 || bls, "NULL arrays");
  return create_hindexed(count, bls, 0, dps, old, out);
}

dt_status dt_create_indexed(int64_t count, const int64_t* bls, const int64_t* d, dt_t old, dt_t* out) {
  CHECK_ARG(old && out, "NULL argument");
  CHECK_ARG(count >= 0, "negative count");
  CHECK_ARG(count == 0 || (bls && d), "NULL arrays");
  std::vector<int64_t> db(d, d + count);
  for (auto& x : db) x *= old->extent();
  return dt_create_hindexed(count, bls, db.data(), old, out);
}

dt_status dt_create_hindexed_block(int64_t count, int64_t blocklen, const int64_t* dps, dt_t old, dt_t* out) {
  CHECK_ARG(count >= 0 && blocklen >= 0, "negative count/blocklen");
  CHECK_ARG(count == 0 || dps, "NULL arrays");
  return create_hindexed(count, nullptr, blocklen, dps, old, out);
}

dt_status dt_create_indexed_block(int64_t count, int64_t blocklen, const int64_t* d, dt_t old, dt_t* out) {
  CHECK_ARG(count >= 0 && blocklen >= 0, "negative count/blocklen");
  CHECK_ARG(count == 0 || d, "NULL arrays");
  CHECK_ARG(old, "NULL argument");
  std::vector<int64_t> db(d, d + count);
  for (auto& x : db) x *= old->extent();
  return create_hindexed(count, nullptr, blocklen, db.data(), old, out);
}

dt_status dt_create_struct(int64_t count, const int64_t* bls, const int64_t* dps, const dt_t* types, dt_t* out) {
  CHECK_ARG(out, "NULL argument");
  CHECK_ARG(count >= 0, "negative count");
  CHECK_ARG(count == 0 || (bls && dps && types), "NULL arrays");
  for (int64_t i = 0; i < count; i++) {
    CHECK_ARG(bls[i] >= 0, "negative blocklen");
    CHECK_ARG(types[i], "NULL component type");
  }
  auto* t = new dt_type_s;
  t->kind = K_STRUCT;
  t->count = count;
  t->bls.assign(bls, bls + count);
  t->dps.assign(dps, dps + count);
  Bounds b;
  for (int64_t i = 0; i < count; i++) {
    t->types.push_back(retain(types[i]));
    if (bls[i] == 0) continue;
    int64_t b0, b1;
    lin_range(bls[i], types[i]->extent(), b0, b1);
    b.add(types[i], dps[i] + b0, dps[i] + b1, bls[i]);
  }
  b.finish(t, true);
  *out = t;
  return DT_OK;
}

dt_status dt_create_subarray(int ndims, const int64_t* sizes, const int64_t* subsizes, const int64_t* starts,
                             int order, dt_t old, dt_t* out) {
  CHECK_ARG(old && out && sizes && subsizes && starts, "NULL argument");
  CHECK_ARG(ndims >= 1 && ndims <= 32, "ndims out of range");
  CHECK_ARG(order == DT_ORDER_C || order == DT_ORDER_FORTRAN, "bad order");
  for (int d = 0; d < ndims; d++) {
    CHECK_ARG(sizes[d] >= 1 && subsizes[d] >= 0 && starts[d] >= 0 && starts[d] + subsizes[d] <= sizes[d],
              "subarray box outside the array");
  }
  auto* t = new dt_type_s;
  t->kind = K_SUBARRAY;
  t->ndims = ndims;
  t->order = order;
  t->sizes.assign(sizes, sizes + ndims);
  t->subsizes.assign(subsizes, subsizes + ndims);
  t->starts.assign(starts, starts + ndims);
  t->old = retain(old);
  // byte stride of each dimension in the full array
  std::vector<int64_t> st(ndims);
  int64_t acc = old->extent();
  if (order == DT_ORDER_C) {
    for (int d = ndims - 1; d >= 0; d--) { st[d] = acc; acc *= sizes[d]; }
  } else {
    for (int d = 0; d < ndims; d++) { st[d] = acc; acc *= sizes[d]; }
  }
  int64_t nel = 1, smin = 0, smax = 0;
  for (int d = 0; d < ndims; d++) {
    nel *= subsizes[d];
    int64_t lo, hi;
    lin_range(subsizes[d], st[d], lo, hi);
    smin += starts[d] * st[d] + lo;
    smax += starts[d] * st[d] + hi;
  }
  Bounds b;
  if (nel > 0) b.add(old, smin, smax, nel);
  b.finish(t, false);
  t->lb = 0;
  t->ub = acc;  // prod(sizes) * extent(old)
  t->has_lb = t->has_ub = true;
  *out = t;
  return DT_OK;
}

dt_status dt_create_resized(dt_t old, int64_t lb, int64_t extent, dt_t* out) {
  CHECK_ARG(old && out, "NULL argument");
  auto* t = new dt_type_s;
  t->kind = K_RESIZED;
  t->old = retain(old);
  t->size = old->size;
  t->align = old->align;
  t->true_lb = old->true_lb;
  t->true_ub = old->true_ub;
  t->lb = lb;
  t->ub = lb + extent;
  t->has_lb = t->has_ub = true;
  *out = t;
  return DT_OK;
}

dt_status dt_get_size(dt_t t, int64_t* size) {
  CHECK_ARG(t && size, "NULL argument");
  *size = t->size;
  return DT_OK;
}
dt_status dt_get_extent(dt_t t, int64_t* lb, int64_t* extent) {
  CHECK_ARG(t && lb && extent, "NULL argument");
  *lb = t->lb;
  *extent = t->extent();
  return DT_OK;
}
dt_status dt_get_true_extent(dt_t t, int64_t* tlb, int64_t* text) {
  CHECK_ARG(t && tlb && text, "NULL argument");
  *tlb = t->true_lb;
  *text = t->true_ub - t->true_lb;
  return DT_OK;
}
dt_status dt_free(dt_t* t) {
  CHECK_ARG(t, "NULL argument");
  if (*t) release(*t);
  *t = nullptr;
  return DT_OK;
}
const char* dt_last_error(void) { return dt::g_err; }
const char* dt_version(void) { return "dt 0.1 (sm_100a)"; }

}  // extern "C"

// ------------------------------------------------------------------ forms
namespace dt {

static void shift_form(Form& f, int64_t s) {
  for (auto& d : f.bd) d += s;
  f.invalidate();
}
static void prepend_regular(Form& f, int64_t cnt, int64_t stride) {
  Level l;
  l.cnt = cnt;
  l.stride = stride;
  f.lv.insert(f.lv.begin(), l);
}
static void prepend_list(Form& f, const std::vector<int64_t>& tab) {
  Level l;
  l.cnt = (int64_t)tab.size();
  l.table = std::make_shared<std::vector<int64_t>>(tab);
  f.lv.insert(f.lv.begin(), l);
}

// merge adjacent blocks, drop empty ones -- in place (a list of 3e7 blocks must not be
// copied again)
static void merge_template(Form& f) {
  size_t w = 0;
  for (size_t i = 0; i < f.bd.size(); i++) {
    if (f.bl[i] == 0) continue;
    if (w > 0 && f.bd[w - 1] + f.bl[w - 1] == f.bd[i]) {
      f.bl[w - 1] += f.bl[i];
    } else {
      f.bd[w] = f.bd[i];
      f.bl[w] = f.bl[i];
      w++;
    }
  }
  f.bd.resize(w);
  f.bl.resize(w);
}

void normalize(Form& f) {
  f.invalidate();
  merge_template(f);
  if (f.bl.empty()) { f.lv.clear(); return; }
  for (auto& l : f.lv)
    if (l.cnt == 0) { f.lv.clear(); f.bd.clear(); f.bl.clear(); return; }
  bool changed = true;
  while (changed) {
    changed = false;
    // list levels that are arithmetic progressions become regular levels
    for (auto& l : f.lv) {
      if (!l.is_list() || l.cnt < 2) continue;
      auto& t = *l.table;
      int64_t st = t[1] - t[0];
      bool ap = true;
      for (int64_t i = 2; i < l.cnt && ap; i++) ap = (t[i] - t[i - 1] == st);
      if (ap) {
        shift_form(f, t[0]);
        l.table.reset();
        l.stride = st;
        changed = true;
      }
    }
    // drop count-1 levels (a list level's single entry is a shift)
    for (size_t i = 0; i < f.lv.size();) {
      if (f.lv[i].cnt == 1) {
        if (f.lv[i].is_list()) shift_form(f, (*f.lv[i].table)[0]);
        f.lv.erase(f.lv.begin() + i);
        changed = true;
      } else {
        i++;
      }
    }
    // innermost regular level over a single block with stride == len: contiguous run
    while (!f.lv.empty() && f.bd.size() == 1 && !f.lv.back().is_list() && f.lv.back().stride == f.bl[0]) {
      f.bl[0] *= f.lv.back().cnt;
      f.lv.pop_back();
      changed = true;
    }
    // adjacent regular levels with stride_outer == cnt_inner * stride_inner
    for (size_t i = 0; i + 1 < f.lv.size(); i++) {
      Level& a = f.lv[i];
      Level& b = f.lv[i + 1];
      if (!a.is_list() && !b.is_list() && a.stride == b.cnt * b.stride) {
        b.cnt *= a.cnt;
        f.lv.erase(f.lv.begin() + i);
        changed = true;
        break;
      }
    }
  }
}

bool expand(const Form& f, std::vector<int64_t>& d, std::vector<int64_t>& l, int64_t cap) {
  d.clear();
  l.clear();
  if (f.bl.empty()) return true;
  const int n = (int)f.lv.size();
  std::vector<int64_t> idx(n, 0);
  int64_t nel = f.nelem();
  if (nel > 0 && (int64_t)f.bl.size() > cap / nel) return false;
  for (int64_t e = 0; e < nel; e++) {
    int64_t disp = 0;
    for (int i = 0; i < n; i++) disp += f.lv[i].contrib(idx[i]);
    for (size_t b = 0; b < f.bd.size(); b++) {
      int64_t x = f.bd[b] + disp;
      if (!d.empty() && d.back() + l.back() == x) l.back() += f.bl[b];
      else { d.push_back(x); l.push_back(f.bl[b]); }
    }
    for (int i = n - 1; i >= 0; i--) {
      if (++idx[i] < f.lv[i].cnt) break;
      idx[i] = 0;
    }
  }
  return true;
}

static int64_t low_pow2(int64_t x) {
  if (x == 0) return 16;
  uint64_t u = (uint64_t)(x < 0 ? -x : x);
  int64_t g = (int64_t)(u & (~u + 1));
  return g > 16 ? 16 : g;
}

// the lowest set bit of an OR over values is the lowest set bit of any of them
static int64_t low_pow2_all(const std::vector<int64_t>& v) {
  uint64_t acc = 0;
  for (int64_t x : v) acc |= (uint64_t)x;  // (two's complement keeps the low bits of |x|)
  return low_pow2((int64_t)acc);
}

int64_t level_granularity(const Form& f) {
  if (f.lvl_gran_cache >= 0) return f.lvl_gran_cache;
  int64_t g = 16;
  for (auto& l : f.lv) {
    if (l.is_list()) g = std::min(g, low_pow2_all(*l.table));
    else g = std::min(g, low_pow2(l.stride));
  }
  f.lvl_gran_cache = g;
  return g;
}

int64_t form_granularity(const Form& f) {
  if (f.gran_cache >= 0) return f.gran_cache;
  int64_t g = 16;
  g = std::min(g, std::min(low_pow2_all(f.bd), low_pow2_all(f.bl)));
  g = std::min(g, level_granularity(f));
  f.gran_cache = g;
  return g;
}

// The flattened form of one instance of t.
static Form build_form(const dt_type_s* t);

static bool is_simple_run(const Form& f, int64_t ext) {
  return f.lv.empty() && f.bd.size() == 1 && f.bl[0] == ext;
}

static bool append_expanded(Form& dst, const Form& src, int64_t shift) {
  std::vector<int64_t> d, l;
  if (!expand(src, d, l, kMaxFlatBlocks - (int64_t)dst.bd.size())) return false;
  for (size_t i = 0; i < d.size(); i++) {
    dst.bd.push_back(d[i] + shift);
    dst.bl.push_back(l[i]);
  }
  return true;
}

struct FlattenError {};

static Form build_form(const dt_type_s* t) {
  Form f;
  switch (t->kind) {
    case K_BASIC:
      f.bd = {0};
      f.bl = {t->size};
      break;
    case K_CONTIG:
    case K_HVECTOR: {
      f = build_form(t->old);
      prepend_regular(f, t->blocklen, t->old->extent());
      prepend_regular(f, t->count, t->stride);
      break;
    }
    case K_HINDEXED: {
      // entries with blocklen 0 contribute nothing; the common cases (a uniform block
      // length, or no zero entries) use the type's arrays as they are -- no filtered
      // copies (first-use cost, f2)
      const std::vector<int64_t>& dps = *t->hdps;
      Form sub = build_form(t->old);
      normalize(sub);
      if (t->count == 0 || sub.empty()) break;
      if (t->blocklen >= 0) {  // hindexed_block: uniform
        if (t->blocklen == 0) break;
        f = sub;
        prepend_regular(f, t->blocklen, t->old->extent());
        Level l;  // the list level shares the type's displacement array
        l.cnt = t->count;
        l.table = t->hdps;
        f.lv.insert(f.lv.begin(), l);
        break;
      }
      const bool all_pos = std::all_of(t->bls.begin(), t->bls.end(), [](int64_t x) { return x > 0; });
      std::vector<int64_t> B, D;
      if (!all_pos) {
        for (int64_t i = 0; i < t->count; i++)
          if (t->bls[i] > 0) { B.push_back(t->bls[i]); D.push_back(dps[i]); }
      }
      const std::vector<int64_t>& Bv = all_pos ? t->bls : B;
      const std::vector<int64_t>& Dv = all_pos ? dps : D;
      if (Bv.empty()) break;
      bool uniform = std::all_of(Bv.begin(), Bv.end(), [&](int64_t x) { return x == Bv[0]; });
      if (uniform) {
        f = sub;
        prepend_regular(f, Bv[0], t->old->extent());
        prepend_list(f, Dv);
      } else if (is_simple_run(sub, t->old->extent())) {
        // indexed of a contiguous element: one block per entry (the triangle C2, the
        // irregular list C5b), adjacent blocks merged in the same pass
        // (one pass; host threads did not pay here: the joined ranges cost a serial copy
        // and concurrent huge-page faults compact memory -- measured slower)
        const int64_t d0 = sub.bd[0], l0 = sub.bl[0];
        huge_reserve(f.bd, Bv.size());
        huge_reserve(f.bl, Bv.size());
        for (size_t i = 0; i < Bv.size(); i++) {
          const int64_t d = Dv[i] + d0, l = Bv[i] * l0;
          if (!f.bd.empty() && f.bd.back() + f.bl.back() == d) f.bl.back() += l;
          else { f.bd.push_back(d); f.bl.push_back(l); }
        }
      } else {
        int64_t e = t->old->extent();
        for (size_t i = 0; i < Bv.size(); i++)
          for (int64_t j = 0; j < Bv[i]; j++)
            if (!append_expanded(f, sub, Dv[i] + j * e)) throw FlattenError();
      }
      break;
    }
    case K_STRUCT: {
      std::vector<int64_t> idx;
      for (int64_t i = 0; i < t->count; i++)
        if (t->bls[i] > 0 && t->types[i]->size > 0) idx.push_back(i);
      if (idx.empty()) break;
      if (idx.size() == 1) {
        int64_t i = idx[0];
        f = build_form(t->types[i]);
        prepend_regular(f, t->bls[i], t->types[i]->extent());
        shift_form(f, t->dps[i]);
        break;
      }
      for (int64_t i : idx) {
        Form sub = build_form(t->types[i]);
        normalize(sub);
        int64_t e = t->types[i]->extent();
        for (int64_t j = 0; j < t->bls[i]; j++)
          if (!append_expanded(f, sub, t->dps[i] + j * e)) throw FlattenError();
      }
      break;
    }
    case K_SUBARRAY: {
      f = build_form(t->old);
      int n = t->ndims;
      std::vector<int64_t> st(n);
      int64_t acc = t->old->extent();
      if (t->order == DT_ORDER_C) {
        for (int d = n - 1; d >= 0; d--) { st[d] = acc; acc *= t->sizes[d]; }
      } else {
        for (int d = 0; d < n; d++) { st[d] = acc; acc *= t->sizes[d]; }
      }
      int64_t base = 0;
      for (int d = 0; d < n; d++) base += t->starts[d] * st[d];
      // prepend from fastest to slowest dimension
      if (t->order == DT_ORDER_C) {
        for (int d = n - 1; d >= 0; d--) prepend_regular(f, t->subsizes[d], st[d]);
      } else {
        for (int d = 0; d < n; d++) prepend_regular(f, t->subsizes[d], st[d]);
      }
      shift_form(f, base);
      break;
    }
    case K_RESIZED:
      f = build_form(t->old);
      break;
    case K_FLAT:
      f = *t->form;
      break;
  }
  normalize(f);
  // keep the kernel's level budget: fold innermost levels into the template
  while ((int)f.lv.size() > kMaxLevels - 1) {
    Level in = f.lv.back();
    f.lv.pop_back();
    Form g;
    g.bd = f.bd;
    g.bl = f.bl;
    g.lv = {in};
    Form h;
    if (!append_expanded(h, g, 0)) throw FlattenError();
    f.bd = h.bd;
    f.bl = h.bl;
    normalize(f);
  }
  return f;
}

bool pipe_list(dt_type_s* t, int64_t* d0, int64_t* l0) {
  if (t->kind != K_HINDEXED || t->blocklen >= 0 || t->count < 2) return false;
  Form sub = build_form(t->old);
  normalize(sub);
  if (!is_simple_run(sub, t->old->extent())) return false;
  *d0 = sub.bd[0];
  *l0 = sub.bl[0];
  return true;
}

void install_form(dt_type_s* t, Form&& f) {
  std::lock_guard<std::mutex> g(t->mu);
  if (!t->form) t->form.reset(new Form(std::move(f)));
}

const Form& get_form(dt_type_s* t) {
  std::lock_guard<std::mutex> g(t->mu);
  if (!t->form) t->form.reset(new Form(build_form(t)));
  return *t->form;
}

static dt_status safe_form(dt_type_s* t, const Form** out) {
  try {
    *out = &get_form(t);
  } catch (FlattenError&) {
    set_error("flattening exceeds %lld blocks", (long long)kMaxFlatBlocks);
    return DT_ERR_NOMEM;
  } catch (std::bad_alloc&) {
    set_error("out of host memory while flattening");
    return DT_ERR_NOMEM;
  }
  return DT_OK;
}

}  // namespace dt

extern "C" {

dt_status dt_get_form(dt_t t, dt_form_info* o) {
  CHECK_ARG(t && o, "NULL argument");
  const Form* f;
  dt_status s = safe_form(t, &f);
  if (s != DT_OK) return s;
  std::memset(o, 0, sizeof(*o));
  o->size = t->size;
  o->lb = t->lb;
  o->extent = t->extent();
  o->true_lb = t->true_lb;
  o->true_extent = t->true_ub - t->true_lb;
  o->nblocks = f->nblocks();
  o->tsize = f->tsize();
  o->nlevels = (int32_t)f->lv.size();
  for (int i = 0; i < o->nlevels && i < 8; i++) {
    o->level_is_list[i] = f->lv[i].is_list();
    o->level_count[i] = f->lv[i].cnt;
    o->level_stride[i] = f->lv[i].stride;
  }
  o->granularity = form_granularity(*f);
  return DT_OK;
}

dt_status dt_flatten(dt_t t, int64_t count, int64_t* disps, int64_t* lens, int64_t max, int64_t* nblocks) {
  CHECK_ARG(t && nblocks && count >= 0 && max >= 0, "bad argument");
  CHECK_ARG(max == 0 || (disps && lens), "NULL output arrays");
  const Form* f;
  dt_status s = safe_form(t, &f);
  if (s != DT_OK) return s;
  if (f->host_missing() && (s = materialize_host(*f, t->devs[0])) != DT_OK) return s;
  Form g = *f;
  if (count != 1) prepend_regular(g, count, t->extent());
  normalize(g);
  std::vector<int64_t> d, l;
  if (!expand(g, d, l, kMaxFlatBlocks)) {
    set_error("dt_flatten: more than %lld blocks", (long long)kMaxFlatBlocks);
    return DT_ERR_NOMEM;
  }
  *nblocks = (int64_t)d.size();
  for (int64_t i = 0; i < (int64_t)d.size() && i < max; i++) {
    disps[i] = d[i];
    lens[i] = l[i];
  }
  return DT_OK;
}

// ------------------------------------------------------------------ serialization
// Wire format (int64 words, native byte order -- homogeneous GPUs, reading A5):
//   magic, version, size, lb, ub, true_lb, true_ub, align, has_lb, has_ub,
//   nlev, nblocks, [cnt, stride, table_len] x nlev, bd[nblocks], bl[nblocks],
//   tables (concatenated, level order).
// This ships a committed layout to a peer rank (direct exchange plans, f1): the
// receiver's flattened form travels, not its constructor tree.
static const int64_t kSerMagic = 0x4454464F524D0001LL;  // "DTFORM" v1

dt_status dt_type_serialize(dt_t t, void* out, size_t* nbytes) {
  CHECK_ARG(t && nbytes, "NULL argument");
  const Form* f;
  dt_status s = safe_form(t, &f);
  if (s != DT_OK) return s;
  if (f->host_missing() && (s = materialize_host(*f, t->devs[0])) != DT_OK) return s;
  std::vector<int64_t> w = {kSerMagic, 1, t->size, t->lb, t->ub, t->true_lb, t->true_ub, t->align,
                            t->has_lb ? 1 : 0, t->has_ub ? 1 : 0, (int64_t)f->lv.size(), (int64_t)f->bd.size()};
  for (auto& l : f->lv) {
    w.push_back(l.cnt);
    w.push_back(l.stride);
    w.push_back(l.is_list() ? (int64_t)l.table->size() : -1);
  }
  w.insert(w.end(), f->bd.begin(), f->bd.end());
  w.insert(w.end(), f->bl.begin(), f->bl.end());
  for (auto& l : f->lv)
    if (l.is_list()) w.insert(w.end(), l.table->begin(), l.table->end());
  const size_t need = w.size() * sizeof(int64_t);
  if (!out) {
    *nbytes = need;
    return DT_OK;
  }
  CHECK_ARG(*nbytes >= need, "buffer too small");
  std::memcpy(out, w.data(), need);
  *nbytes = need;
  return DT_OK;
}

dt_status dt_type_deserialize(const void* in, size_t nbytes, dt_t* out) {
  CHECK_ARG(in && out, "NULL argument");
  CHECK_ARG(nbytes % 8 == 0 && nbytes >= 12 * 8, "truncated type blob");
  const size_t nw = nbytes / 8;
  std::vector<int64_t> w(nw);
  std::memcpy(w.data(), in, nbytes);
  CHECK_ARG(w[0] == kSerMagic && w[1] == 1, "not a serialized dt type");
  const int64_t nlev = w[10], nb = w[11];
  CHECK_ARG(nlev >= 0 && nlev < kMaxLevels && nb >= 0, "corrupt type blob");
  size_t k = 12;
  CHECK_ARG(k + 3 * (size_t)nlev + 2 * (size_t)nb <= nw, "truncated type blob");
  std::unique_ptr<Form> f(new Form);
  std::vector<int64_t> tl;
  for (int64_t i = 0; i < nlev; i++) {
    Level l;
    l.cnt = w[k++];
    l.stride = w[k++];
    tl.push_back(w[k++]);
    f->lv.push_back(l);
  }
  f->bd.assign(w.begin() + k, w.begin() + k + nb);
  k += nb;
  f->bl.assign(w.begin() + k, w.begin() + k + nb);
  k += nb;
  for (int64_t i = 0; i < nlev; i++) {
    if (tl[i] < 0) continue;
    CHECK_ARG(tl[i] == f->lv[i].cnt && k + (size_t)tl[i] <= nw, "truncated type blob");
    f->lv[i].table = std::make_shared<std::vector<int64_t>>(w.begin() + k, w.begin() + k + tl[i]);
    f->lv[i].stride = 0;
    k += tl[i];
  }
  CHECK_ARG(k == nw, "trailing bytes in type blob");
  auto* t = new dt_type_s;
  t->kind = K_FLAT;
  t->size = w[2];
  t->lb = w[3];
  t->ub = w[4];
  t->true_lb = w[5];
  t->true_ub = w[6];
  t->align = w[7];
  t->has_lb = w[8] != 0;
  t->has_ub = w[9] != 0;
  t->form = std::move(f);
  *out = t;
  return DT_OK;
}

}  // extern "C"
