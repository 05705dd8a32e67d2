/*
 * oracle.c — plain, slow, obviously-correct CPU oracle for MPI datatype pack/unpack.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h): loaded by tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs; never by the product path.
 *
 * Paper passages followed (PAPER.md, Wu et al. HPDC'16):
 *   - constructors contiguous / vector / indexed / struct: [L14:c1262 §3]
 *   - pack = gather the typemap's bytes into a contiguous buffer, unpack = the
 *     inverse scatter; the contiguous buffer is "the destination for the pack
 *     operation, and the source for the unpack" [L16:c5201 §3.2]
 *   - pack/unpack restart from a position ("converts only a part of the
 *     datatype", [L18:c1430 §3.2]; fragment index [L20:c1815 §4.1]) -> pos/len.
 *   - sub-matrix (vector) and triangle (indexed) workloads [L22:c1966], [L22:c2839 §5.1].
 * MPI-3.1 §4.1 defines each constructor's typemap; bounds per §4.1.6 with the
 * readings R-eps (alignment padding only for struct) and R-markers (explicit
 * lb/ub markers of resized/subarray copies win over data entries), DESIGN.md.
 *
 * Method: each type is a constructor tree.  walk() enumerates the basic
 * elements in typemap order by literally running the constructor loops.  The
 * only shortcut is skipping a subtree whose `size` bytes lie entirely before
 * the requested stream position (each subtree contributes exactly size bytes).
 */
#include "oracle.h"
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

enum { K_BASIC, K_CONTIG, K_HVECTOR, K_HINDEXED, K_STRUCT, K_SUBARRAY, K_RESIZED };

struct or_type {
  int refcnt;
  int kind;
  int basic;                 /* K_BASIC: basic kind */
  int64_t count;             /* CONTIG/HVECTOR/HINDEXED/STRUCT */
  int64_t blocklen;          /* HVECTOR */
  int64_t stride;            /* HVECTOR, bytes */
  int64_t* bls;              /* HINDEXED/STRUCT blocklens */
  int64_t* dps;              /* HINDEXED/STRUCT displacements, bytes */
  or_type** types;           /* STRUCT */
  int ndims, order;          /* SUBARRAY */
  int64_t *sizes, *subsizes, *starts;
  or_type* old;
  /* bounds, computed eagerly at construction */
  int64_t size, lb, ub, true_lb, true_ub, nentries, align;
  int has_lb, has_ub;
};

static const int64_t basic_size[8] = {1, 1, 1, 2, 4, 8, 4, 8};

static or_type* new_type(int kind) {
  or_type* t = (or_type*)calloc(1, sizeof(or_type));
  t->refcnt = 1;
  t->kind = kind;
  return t;
}
static or_type* ref(or_type* t) { t->refcnt++; return t; }
static int64_t ext(const or_type* t) { return t->ub - t->lb; }
static int64_t* dup64(const int64_t* a, int64_t n) {
  int64_t* r = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  if (n > 0) memcpy(r, a, sizeof(int64_t) * (size_t)n);
  return r;
}

/* ---- bounds accumulation over the copies a constructor makes (MPI-3.1 §4.1.6) ----
 * A copy of T shifted by s contributes:
 *   lb: marker s+lb(T) if T carries an lb marker, else (if T has data) s+lb(T);
 *   ub: marker s+ub(T) if T carries a ub marker, else (if T has data) s+ub(T);
 *   true bounds: s+true_lb(T), s+true_ub(T) if T has data.
 * If any copy contributed a marker, only markers count (R-markers). */
typedef struct {
  int any_lbm, any_ubm, any_data;
  int64_t lbm, ubm, dlb, dub, tlb, tub, size, nent, align;
} bacc;

static void bacc_init(bacc* a) { memset(a, 0, sizeof(*a)); a->align = 1; }
static void bacc_copy(bacc* a, const or_type* T, int64_t s) {
  if (T->has_lb) { if (!a->any_lbm || s + T->lb < a->lbm) a->lbm = s + T->lb; a->any_lbm = 1; }
  if (T->has_ub) { if (!a->any_ubm || s + T->ub > a->ubm) a->ubm = s + T->ub; a->any_ubm = 1; }
  if (T->size > 0) {
    if (!a->any_data) { a->dlb = s + T->lb; a->dub = s + T->ub; a->tlb = s + T->true_lb; a->tub = s + T->true_ub; }
    else {
      if (s + T->lb < a->dlb) a->dlb = s + T->lb;
      if (s + T->ub > a->dub) a->dub = s + T->ub;
      if (s + T->true_lb < a->tlb) a->tlb = s + T->true_lb;
      if (s + T->true_ub > a->tub) a->tub = s + T->true_ub;
    }
    a->any_data = 1;
  }
  a->size += T->size;
  a->nent += T->nentries;
  if (T->align > a->align) a->align = T->align;
}
static void bacc_finish(bacc* a, or_type* t, int is_struct) {
  t->size = a->size;
  t->nentries = a->nent;
  t->align = a->align;
  t->has_lb = a->any_lbm;
  t->has_ub = a->any_ubm;
  t->lb = a->any_lbm ? a->lbm : (a->any_data ? a->dlb : 0);
  t->ub = a->any_ubm ? a->ubm : (a->any_data ? a->dub : 0);
  if (is_struct && !a->any_ubm && a->any_data) {
    /* R-eps: struct rounds its extent up to a multiple of the largest basic alignment */
    int64_t e = t->ub - t->lb;
    int64_t r = ((e % a->align) + a->align) % a->align;
    if (r) t->ub += a->align - r;
  }
  t->true_lb = a->any_data ? a->tlb : 0;
  t->true_ub = a->any_data ? a->tub : 0;
}

or_type* or_basic(int kind) {
  if (kind < 0 || kind > 7) return NULL;
  or_type* t = new_type(K_BASIC);
  t->basic = kind;
  t->size = basic_size[kind];
  t->lb = 0; t->ub = t->size;
  t->true_lb = 0; t->true_ub = t->size;
  t->nentries = 1;
  t->align = basic_size[kind];
  return t;
}

/* MPI: contiguous(n, T) — n copies of T at i*extent(T) */
or_type* or_contiguous(int64_t count, or_type* old) {
  or_type* t = new_type(K_CONTIG);
  t->count = count; t->old = ref(old);
  bacc a; bacc_init(&a);
  for (int64_t i = 0; i < count; i++) bacc_copy(&a, old, i * ext(old));
  bacc_finish(&a, t, 0);
  return t;
}

/* MPI: hvector(c, b, s, T) — for i<c, j<b: T at i*s + j*extent(T) (s in bytes) */
or_type* or_hvector(int64_t count, int64_t blocklen, int64_t stride, or_type* old) {
  or_type* t = new_type(K_HVECTOR);
  t->count = count; t->blocklen = blocklen; t->stride = stride; t->old = ref(old);
  bacc a; bacc_init(&a);
  for (int64_t i = 0; i < count; i++)
    for (int64_t j = 0; j < blocklen; j++) bacc_copy(&a, old, i * stride + j * ext(old));
  bacc_finish(&a, t, 0);
  return t;
}
/* MPI: vector(c, b, s, T) == hvector(c, b, s*extent(T), T) */
or_type* or_vector(int64_t count, int64_t blocklen, int64_t stride, or_type* old) {
  return or_hvector(count, blocklen, stride * ext(old), old);
}

/* MPI: hindexed(c, B[], D[], T) — for i<c, j<B[i]: T at D[i] + j*extent(T) (D in bytes) */
or_type* or_hindexed(int64_t count, const int64_t* bls, const int64_t* dps, or_type* old) {
  or_type* t = new_type(K_HINDEXED);
  t->count = count; t->bls = dup64(bls, count); t->dps = dup64(dps, count); t->old = ref(old);
  bacc a; bacc_init(&a);
  for (int64_t i = 0; i < count; i++)
    for (int64_t j = 0; j < bls[i]; j++) bacc_copy(&a, old, dps[i] + j * ext(old));
  bacc_finish(&a, t, 0);
  return t;
}
/* MPI: indexed(c, B[], D[], T) == hindexed with D[i]*extent(T) */
or_type* or_indexed(int64_t count, const int64_t* bls, const int64_t* d, or_type* old) {
  int64_t* db = dup64(d, count);
  for (int64_t i = 0; i < count; i++) db[i] = d[i] * ext(old);
  or_type* t = or_hindexed(count, bls, db, old);
  free(db);
  return t;
}
or_type* or_hindexed_block(int64_t count, int64_t blocklen, const int64_t* dps, or_type* old) {
  int64_t* b = (int64_t*)malloc(sizeof(int64_t) * (size_t)(count > 0 ? count : 1));
  for (int64_t i = 0; i < count; i++) b[i] = blocklen;
  or_type* t = or_hindexed(count, b, dps, old);
  free(b);
  return t;
}
or_type* or_indexed_block(int64_t count, int64_t blocklen, const int64_t* d, or_type* old) {
  int64_t* b = (int64_t*)malloc(sizeof(int64_t) * (size_t)(count > 0 ? count : 1));
  for (int64_t i = 0; i < count; i++) b[i] = blocklen;
  or_type* t = or_indexed(count, b, d, old);
  free(b);
  return t;
}

/* MPI: struct(c, B[], D[], T[]) — for i<c, j<B[i]: T[i] at D[i] + j*extent(T[i]) */
or_type* or_struct(int64_t count, const int64_t* bls, const int64_t* dps, or_type* const* types) {
  or_type* t = new_type(K_STRUCT);
  t->count = count; t->bls = dup64(bls, count); t->dps = dup64(dps, count);
  t->types = (or_type**)malloc(sizeof(or_type*) * (size_t)(count > 0 ? count : 1));
  bacc a; bacc_init(&a);
  for (int64_t i = 0; i < count; i++) {
    t->types[i] = ref(types[i]);
    for (int64_t j = 0; j < bls[i]; j++) bacc_copy(&a, types[i], dps[i] + j * ext(types[i]));
  }
  bacc_finish(&a, t, 1);
  return t;
}

/* MPI: subarray(n, sizes, subsizes, starts, order, T): the elements of the
 * sub-box, enumerated in array order (C: last index fastest; Fortran: first
 * fastest), at the linear array offset of (starts+idx) times extent(T); the
 * result is resized to lb = 0, extent = prod(sizes)*extent(T). */
static int64_t sub_linear(const or_type* t, const int64_t* idx) {
  int64_t lin = 0;
  if (t->order == 0) {
    for (int d = 0; d < t->ndims; d++) lin = lin * t->sizes[d] + (t->starts[d] + idx[d]);
  } else {
    for (int d = t->ndims - 1; d >= 0; d--) lin = lin * t->sizes[d] + (t->starts[d] + idx[d]);
  }
  return lin;
}
/* advance the odometer idx[] in array order; returns 0 when wrapped */
static int sub_next(const or_type* t, int64_t* idx) {
  if (t->order == 0) {
    for (int d = t->ndims - 1; d >= 0; d--) { if (++idx[d] < t->subsizes[d]) return 1; idx[d] = 0; }
  } else {
    for (int d = 0; d < t->ndims; d++) { if (++idx[d] < t->subsizes[d]) return 1; idx[d] = 0; }
  }
  return 0;
}
or_type* or_subarray(int ndims, const int64_t* sizes, const int64_t* subsizes, const int64_t* starts,
                     int order, or_type* old) {
  or_type* t = new_type(K_SUBARRAY);
  t->ndims = ndims; t->order = order; t->old = ref(old);
  t->sizes = dup64(sizes, ndims); t->subsizes = dup64(subsizes, ndims); t->starts = dup64(starts, ndims);
  bacc a; bacc_init(&a);
  int64_t nel = 1, tot = 1;
  for (int d = 0; d < ndims; d++) { nel *= subsizes[d]; tot *= sizes[d]; }
  if (nel > 0) {
    int64_t idx[32] = {0};
    do { bacc_copy(&a, old, sub_linear(t, idx) * ext(old)); } while (sub_next(t, idx));
  }
  bacc_finish(&a, t, 0);
  t->lb = 0; t->ub = tot * ext(old); t->has_lb = 1; t->has_ub = 1;
  return t;
}

/* MPI: resized(T, lb, extent) — same typemap, explicit lb/ub markers */
or_type* or_resized(or_type* old, int64_t lb, int64_t extent) {
  or_type* t = new_type(K_RESIZED);
  t->old = ref(old);
  t->size = old->size; t->nentries = old->nentries; t->align = old->align;
  t->true_lb = old->true_lb; t->true_ub = old->true_ub;
  t->lb = lb; t->ub = lb + extent; t->has_lb = 1; t->has_ub = 1;
  return t;
}

void or_free(or_type* t) {
  if (!t || --t->refcnt > 0) return;
  if (t->old) or_free(t->old);
  if (t->types) { for (int64_t i = 0; i < t->count; i++) or_free(t->types[i]); free(t->types); }
  free(t->bls); free(t->dps); free(t->sizes); free(t->subsizes); free(t->starts);
  free(t);
}

void or_info(const or_type* t, int64_t* out) {
  out[0] = t->size; out[1] = t->lb; out[2] = t->ub; out[3] = t->ub - t->lb;
  out[4] = t->true_lb; out[5] = t->true_ub; out[6] = t->nentries;
}

/* ---------------- the typemap walk ---------------- */
typedef struct visitor visitor;
struct visitor {
  void (*fn)(visitor* v, int kind, int64_t disp);
  int64_t cursor;   /* stream position of the next element */
  int64_t pos, end; /* requested window [pos, end) */
  int done;
  /* payload */
  const uint8_t* src; uint8_t* dst;   /* pack: src = origin, dst = out; unpack: src = packed, dst = origin */
  int64_t* kinds; int64_t* disps; int64_t max;
  const int64_t* ps; int64_t np, ip; int64_t* addr;
};

static void walk(const or_type* t, int64_t shift, visitor* v) {
  if (v->done) return;
  if (v->cursor + t->size <= v->pos) { v->cursor += t->size; return; } /* subtree entirely before pos */
  switch (t->kind) {
  case K_BASIC:
    v->fn(v, t->basic, shift);
    v->cursor += t->size;
    if (v->cursor >= v->end) v->done = 1;
    break;
  case K_CONTIG:
    for (int64_t i = 0; i < t->count && !v->done; i++) walk(t->old, shift + i * ext(t->old), v);
    break;
  case K_HVECTOR:
    for (int64_t i = 0; i < t->count && !v->done; i++)
      for (int64_t j = 0; j < t->blocklen && !v->done; j++)
        walk(t->old, shift + i * t->stride + j * ext(t->old), v);
    break;
  case K_HINDEXED:
    for (int64_t i = 0; i < t->count && !v->done; i++)
      for (int64_t j = 0; j < t->bls[i] && !v->done; j++)
        walk(t->old, shift + t->dps[i] + j * ext(t->old), v);
    break;
  case K_STRUCT:
    for (int64_t i = 0; i < t->count && !v->done; i++)
      for (int64_t j = 0; j < t->bls[i] && !v->done; j++)
        walk(t->types[i], shift + t->dps[i] + j * ext(t->types[i]), v);
    break;
  case K_SUBARRAY: {
    int64_t nel = 1;
    for (int d = 0; d < t->ndims; d++) nel *= t->subsizes[d];
    if (nel == 0) break;
    int64_t idx[32] = {0};
    do { walk(t->old, shift + sub_linear(t, idx) * ext(t->old), v); } while (!v->done && sub_next(t, idx));
    break;
  }
  case K_RESIZED:
    walk(t->old, shift, v);
    break;
  }
}

/* walk `count` instances; instance k rooted at k*extent */
static void walk_count(const or_type* t, int64_t count, visitor* v) {
  v->done = (v->pos >= v->end);
  v->cursor = 0;
  if (t->size > 0 && v->pos > 0) {          /* skip whole instances before pos */
    int64_t k0 = v->pos / t->size;
    v->cursor = k0 * t->size;
    for (int64_t k = k0; k < count && !v->done; k++) walk(t, k * ext(t), v);
    return;
  }
  for (int64_t k = 0; k < count && !v->done; k++) walk(t, k * ext(t), v);
}

static void fn_pack(visitor* v, int kind, int64_t disp) {
  int64_t sz = basic_size[kind];
  for (int64_t b = 0; b < sz; b++) {
    int64_t p = v->cursor + b;
    if (p >= v->pos && p < v->end) v->dst[p - v->pos] = v->src[disp + b];
  }
}
static void fn_unpack(visitor* v, int kind, int64_t disp) {
  int64_t sz = basic_size[kind];
  for (int64_t b = 0; b < sz; b++) {
    int64_t p = v->cursor + b;
    if (p >= v->pos && p < v->end) v->dst[disp + b] = v->src[p - v->pos];
  }
}
static void fn_typemap(visitor* v, int kind, int64_t disp) {
  if (v->ip < v->max) { v->kinds[v->ip] = kind; v->disps[v->ip] = disp; }
  v->ip++;
}
static void fn_addr(visitor* v, int kind, int64_t disp) {
  int64_t sz = basic_size[kind];
  while (v->ip < v->np && v->ps[v->ip] < v->cursor + sz) {
    if (v->ps[v->ip] >= v->cursor) v->addr[v->ip] = disp + (v->ps[v->ip] - v->cursor);
    else v->addr[v->ip] = INT64_MIN;   /* unsorted / before window: not reachable */
    v->ip++;
  }
  if (v->ip >= v->np) v->done = 1;
}

static int64_t clip(const or_type* t, int64_t count, int64_t pos, int64_t len) {
  int64_t total = count * t->size;
  if (pos >= total || len <= 0 || pos < 0) return 0;
  return len < total - pos ? len : total - pos;
}

int64_t or_typemap(const or_type* t, int64_t* kinds, int64_t* disps, int64_t max) {
  visitor v; memset(&v, 0, sizeof(v));
  v.fn = fn_typemap; v.kinds = kinds; v.disps = disps; v.max = max;
  v.pos = 0; v.end = INT64_MAX;
  walk(t, 0, &v);
  return v.ip;
}

int64_t or_pack(const or_type* t, int64_t count, const uint8_t* origin, uint8_t* out, int64_t pos, int64_t len) {
  int64_t n = clip(t, count, pos, len);
  if (n == 0) return 0;
  visitor v; memset(&v, 0, sizeof(v));
  v.fn = fn_pack; v.src = origin; v.dst = out; v.pos = pos; v.end = pos + n;
  walk_count(t, count, &v);
  return n;
}

int64_t or_unpack(const or_type* t, int64_t count, const uint8_t* packed, uint8_t* origin, int64_t pos, int64_t len) {
  int64_t n = clip(t, count, pos, len);
  if (n == 0) return 0;
  visitor v; memset(&v, 0, sizeof(v));
  v.fn = fn_unpack; v.src = packed; v.dst = origin; v.pos = pos; v.end = pos + n;
  walk_count(t, count, &v);
  return n;
}

int64_t or_addr_of(const or_type* t, int64_t count, const int64_t* ps, int64_t n, int64_t* out) {
  if (n <= 0) return 0;
  visitor v; memset(&v, 0, sizeof(v));
  v.fn = fn_addr; v.ps = ps; v.np = n; v.addr = out;
  for (int64_t i = 0; i < n; i++) out[i] = INT64_MIN;
  v.pos = ps[0]; v.end = count * t->size;
  if (v.pos < 0) v.pos = 0;
  walk_count(t, count, &v);
  return v.ip;
}

/* ---- multithreaded timing mode: equal byte ranges, each thread seeks independently ---- */
typedef struct { const or_type* t; int64_t count; const uint8_t* a; uint8_t* b; int64_t pos, len; int unpack; } job;
static void* run_job(void* p) {
  job* j = (job*)p;
  if (j->unpack) or_unpack(j->t, j->count, j->a, j->b, j->pos, j->len);
  else or_pack(j->t, j->count, j->a, j->b, j->pos, j->len);
  return NULL;
}
static int64_t run_mt(const or_type* t, int64_t count, const uint8_t* a, uint8_t* b, int64_t pos, int64_t len,
                      int nthreads, int unpack) {
  int64_t n = clip(t, count, pos, len);
  if (n == 0) return 0;
  if (nthreads < 1) nthreads = 1;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)nthreads);
  job* jobs = (job*)malloc(sizeof(job) * (size_t)nthreads);
  int64_t per = (n + nthreads - 1) / nthreads;
  for (int i = 0; i < nthreads; i++) {
    int64_t s = (int64_t)i * per, e = s + per > n ? n : s + per;
    jobs[i].t = t; jobs[i].count = count; jobs[i].unpack = unpack;
    jobs[i].pos = pos + s; jobs[i].len = e > s ? e - s : 0;
    if (unpack) { jobs[i].a = a + s; jobs[i].b = b; }   /* packed slice s.. goes to its addresses */
    else { jobs[i].a = a; jobs[i].b = b + s; }
    pthread_create(&th[i], NULL, run_job, &jobs[i]);
  }
  for (int i = 0; i < nthreads; i++) pthread_join(th[i], NULL);
  free(th); free(jobs);
  return n;
}
int64_t or_pack_mt(const or_type* t, int64_t count, const uint8_t* origin, uint8_t* out, int64_t pos, int64_t len, int nthreads) {
  return run_mt(t, count, origin, out, pos, len, nthreads, 0);
}
int64_t or_unpack_mt(const or_type* t, int64_t count, const uint8_t* packed, uint8_t* origin, int64_t pos, int64_t len, int nthreads) {
  return run_mt(t, count, packed, origin, pos, len, nthreads, 1);
}
