/*
 * oracle.h — CPU oracle for MPI-derived-datatype pack/unpack.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product
 * (paper_conf_hpdc_wubvjd16_b200/, libdt.so) never links, includes or calls it,
 * and it shares no code, header, table or helper with the CUDA path.
 *
 * What it computes: the plain MPI typemap definition of pack/unpack that the
 * paper's GPU datatype engine reproduces "for any MPI datatype"
 * (PAPER.md [L18:c1021 §3.2]); constructors named in [L14:c1262 §3]; the pack
 * result is the concatenation, in typemap order, of the basic elements of
 * `count` instances (instance k rooted at origin + k*extent).  Semantics of the
 * constructors and of lb/ub/extent follow MPI-3.1 §4.1 (which the paper relies
 * on without restating); the readings taken where the standard is
 * implementation-defined are listed in DESIGN.md §Readings (R-eps, R-markers).
 *
 * Every type is a tree of constructor nodes; the typemap is enumerated by a
 * plain recursive walk (oracle.c: walk()) — no flattening, merging, blocking
 * or reordering.
 */
#ifndef DT_ORACLE_H
#define DT_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct or_type or_type;

/* basic kinds: 0 BYTE, 1 CHAR, 2 INT8, 3 INT16, 4 INT32, 5 INT64, 6 FLOAT, 7 DOUBLE */
or_type* or_basic(int kind);
or_type* or_contiguous(int64_t count, or_type* old);
or_type* or_vector(int64_t count, int64_t blocklen, int64_t stride_elems, or_type* old);
or_type* or_hvector(int64_t count, int64_t blocklen, int64_t stride_bytes, or_type* old);
or_type* or_indexed(int64_t count, const int64_t* blocklens, const int64_t* displs_elems, or_type* old);
or_type* or_hindexed(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes, or_type* old);
or_type* or_indexed_block(int64_t count, int64_t blocklen, const int64_t* displs_elems, or_type* old);
or_type* or_hindexed_block(int64_t count, int64_t blocklen, const int64_t* displs_bytes, or_type* old);
or_type* or_struct(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes, or_type* const* types);
or_type* or_subarray(int ndims, const int64_t* sizes, const int64_t* subsizes, const int64_t* starts,
                     int order /*0=C,1=Fortran*/, or_type* old);
or_type* or_resized(or_type* old, int64_t lb, int64_t extent);
void     or_free(or_type* t);

/* out[0..6] = size, lb, ub, extent, true_lb, true_ub, nentries(number of basic elements) */
void     or_info(const or_type* t, int64_t* out);

/* Enumerate the typemap: kinds[i], disps[i] for i < min(max, nentries).  Returns nentries. */
int64_t  or_typemap(const or_type* t, int64_t* kinds, int64_t* disps, int64_t max);

/* Pack stream bytes [pos, pos+len) of `count` instances rooted at `origin`
 * (instance k at origin + k*extent) into out[0 .. ).  Returns bytes written
 * = min(len, count*size - pos) (0 if pos >= total). */
int64_t  or_pack(const or_type* t, int64_t count, const uint8_t* origin, uint8_t* out, int64_t pos, int64_t len);
/* Inverse: write packed[0..) (stream bytes [pos, pos+len)) to their typemap addresses. */
int64_t  or_unpack(const or_type* t, int64_t count, const uint8_t* packed, uint8_t* origin, int64_t pos, int64_t len);
/* Multithreaded timing mode: split [pos,pos+len) into nthreads equal ranges, one pthread each. */
int64_t  or_pack_mt(const or_type* t, int64_t count, const uint8_t* origin, uint8_t* out, int64_t pos, int64_t len, int nthreads);
int64_t  or_unpack_mt(const or_type* t, int64_t count, const uint8_t* packed, uint8_t* origin, int64_t pos, int64_t len, int nthreads);
/* Address (relative to origin) of stream byte positions ps[i] (sorted ascending); out[i]. */
int64_t  or_addr_of(const or_type* t, int64_t count, const int64_t* ps, int64_t n, int64_t* out);

#ifdef __cplusplus
}
#endif
#endif
