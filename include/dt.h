/*
 * dt.h — C-ABI of the B200-native MPI-derived-datatype engine (libdt.so).
 *
 * Implements the hot path of Wu, Bosilca, vandeVaart, Jeaugey, Dongarra,
 * "GPU-Aware Non-contiguous Data Movement In Open MPI", HPDC'16:
 *   - describing a non-contiguous GPU-resident layout once with MPI
 *     constructors and committing it ([L10:c3576 §1], [L10:c4029 §1],
 *     constructors [L14:c1262 §3]);
 *   - packing / unpacking it on the GPU on a caller stream ([L16:c2435 §3.1]:
 *     "launched in a dedicated CUDA stream ... complete after a
 *     synchronization with the stream"), for any datatype ([L18:c1021 §3.2]);
 *   - resuming a pack/unpack at a byte position so a pipeline can stop and
 *     restart per fragment ([L18:c1430 §3.2], fragment index [L20:c1815 §4.1]);
 *   - moving data between GPU ranks with a pipelined pack -> transfer -> unpack
 *     ([L18:c4394]-[L18:c5513 §4.1], [L20:c2905]-[L20:c4255 §4.1]).
 *
 * Conventions (all entry points):
 *   - Integer widths follow MPI-4 "large count": int64_t counts, byte
 *     displacements, sizes.  Displacements may be negative (MPI).
 *   - No torch / C++ types cross this boundary: plain handles, integers,
 *     host pointers (H) and device pointers (D).  Streams are cudaStream_t
 *     passed as void* (0 = legacy default stream).
 *   - Every function returns a dt_status; none aborts.  dt_last_error()
 *     returns a thread-local message for the last non-DT_OK status.
 *   - There is NO CPU fallback: buffers handed to pack/unpack/sendrecv must be
 *     device memory of the current device (DT_ERR_ARG otherwise).
 */
#ifndef DT_H
#define DT_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct dt_type_s* dt_t;      /* opaque; refcounted; immutable after commit            */
typedef struct dt_comm_s* dt_comm_t; /* opaque; one per (process, device, peer set)            */

typedef enum {
  DT_OK = 0,
  DT_ERR_ARG = 1,           /* bad argument (NULL, negative count, host pointer, bad rank ...)  */
  DT_ERR_NOT_COMMITTED = 2, /* pack/unpack/sendrecv on a type that was never dt_commit()ed      */
  DT_ERR_OVERLAP = 3,       /* unpack into a typemap whose entries overlap (MPI: erroneous)     */
  DT_ERR_TRUNCATE = 4,      /* sendrecv: send bytes > receive capacity                          */
  DT_ERR_CUDA = 5,          /* a CUDA runtime call failed (message in dt_last_error)            */
  DT_ERR_NCCL = 6,          /* NCCL unavailable or a NCCL call failed                           */
  DT_ERR_NOMEM = 7,         /* host/device allocation failed or flattening exceeded its cap     */
  DT_ERR_TIMEOUT = 8,       /* a bounded device-side wait for a peer flag expired               */
  DT_ERR_UNSUPPORTED = 9    /* valid request this build does not implement                      */
} dt_status;

typedef enum { DT_BYTE = 0, DT_CHAR, DT_INT8, DT_INT16, DT_INT32, DT_INT64, DT_FLOAT, DT_DOUBLE } dt_basic;
enum { DT_ORDER_C = 0, DT_ORDER_FORTRAN = 1 };

/* ------------------------------------------------------------------ types
 * Constructors follow MPI-3.1 §4.1 (the paper names them at [L14:c1262 §3]
 * and relies on the standard for their meaning).  On success *out receives a
 * new handle holding one reference; components are referenced, so freeing a
 * component afterwards is safe (as in MPI).  Bounds: lb/ub/extent per
 * MPI-3.1 §4.1.6 with the readings R-eps (alignment padding only for struct)
 * and R-markers (explicit lb/ub of resized/subarray win), DESIGN.md.
 * Errors: DT_ERR_ARG for NULL pointers, negative counts/blocklens, ndims<1,
 * subarray boxes outside sizes, unknown basic kind. */
dt_t      dt_basic_type(dt_basic k);                       /* predefined, never freed; NULL if k invalid */
dt_status dt_create_contiguous(int64_t count, dt_t old, dt_t* out);
/* stride in elements of extent(old) (start-to-start, reading A16) */
dt_status dt_create_vector(int64_t count, int64_t blocklen, int64_t stride_elems, dt_t old, dt_t* out);
dt_status dt_create_hvector(int64_t count, int64_t blocklen, int64_t stride_bytes, dt_t old, dt_t* out);
/* blocklens[i] elements at displs[i] (H arrays of length count, copied) */
dt_status dt_create_indexed(int64_t count, const int64_t* blocklens, const int64_t* displs_elems, dt_t old, dt_t* out);
dt_status dt_create_hindexed(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes, dt_t old, dt_t* out);
dt_status dt_create_indexed_block(int64_t count, int64_t blocklen, const int64_t* displs_elems, dt_t old, dt_t* out);
dt_status dt_create_hindexed_block(int64_t count, int64_t blocklen, const int64_t* displs_bytes, dt_t old, dt_t* out);
dt_status dt_create_struct(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes, const dt_t* types,
                           dt_t* out);
/* sizes/subsizes/starts: H arrays of ndims; order DT_ORDER_C (last index fastest) or
 * DT_ORDER_FORTRAN; result has lb 0 and extent prod(sizes)*extent(old). */
dt_status dt_create_subarray(int ndims, const int64_t* sizes, const int64_t* subsizes, const int64_t* starts,
                             int order, dt_t old, dt_t* out);
dt_status dt_create_resized(dt_t old, int64_t lb, int64_t extent, dt_t* out);

/* Flatten the type into its GPU descriptor (strided levels + (disp,len) block
 * template, [L16:c1326 §3], DEVs [L16:c5201 §3.2]) and upload it to the CURRENT
 * device, where a device prefix scan (warp shuffles) computes the block
 * offsets; the descriptor is cached on the type ([L18:c1649 §3.2]).
 * Idempotent; may be called again from another device.  Stream: legacy
 * default; returns after the upload completed.  Errors: DT_ERR_NOMEM if the
 * flattened form exceeds its cap, DT_ERR_CUDA. */
dt_status dt_commit(dt_t t);
dt_status dt_get_size(dt_t t, int64_t* size);
dt_status dt_get_extent(dt_t t, int64_t* lb, int64_t* extent);
dt_status dt_get_true_extent(dt_t t, int64_t* true_lb, int64_t* true_extent);
/* Drops one reference and sets *t = NULL.  Predefined types are ignored. */
dt_status dt_free(dt_t* t);

/* ------------------------------------------------------------------ pack / unpack
 * The packed stream of `count` instances of t rooted at `origin` (instance k
 * at origin + k*extent(t); typemap displacement d at origin + k*extent + d,
 * d may be negative) is the concatenation in typemap order of the bytes of
 * every basic element (native representation, no conversion: reading A5).
 *
 * dt_pack: copies stream bytes [pos, pos + *len) from the layout at `origin`
 *   (D, read-only) into `packed` (D): packed[0] receives stream byte pos.
 * dt_unpack: writes `packed` (D; stream bytes [pos, pos + *len)) to their
 *   typemap addresses under `origin` (D); bytes outside the typemap are never
 *   written.  Rejects overlapping typemaps with DT_ERR_OVERLAP (reading A9).
 * In: *len = maximum bytes.  Out: *len = min(*len, count*size - pos), 0 if
 * pos >= count*size.  pos is byte-granular (reading A7).  Both are
 * asynchronous on `stream` (void* = cudaStream_t) and complete in stream
 * order; no host synchronisation.  Errors: DT_ERR_NOT_COMMITTED,
 * DT_ERR_ARG (NULL, negative count/pos, host pointer), DT_ERR_CUDA. */
dt_status dt_pack(dt_t t, int64_t count, const void* origin, void* packed, int64_t pos, int64_t* len, void* stream);
dt_status dt_unpack(dt_t t, int64_t count, const void* packed, void* origin, int64_t pos, int64_t* len, void* stream);

/* Same operations on HOST buffers: page-locked (pinned, device-mapped) buffers
 * are read and written by the pack/unpack kernel itself over the host link
 * (zero-copy: only the typemap's bytes and the packed stream cross it; unpack
 * writes only typemap bytes, so host gap bytes stay untouched); pageable
 * buffers are staged through device memory on `stream` (H2D of the layout
 * span, GPU pack/unpack, D2H of the result; DT_HOST_STAGED=1 forces this).
 * Synchronises the stream before returning.  This is the end-to-end entry
 * point a host user calls; all byte movement happens in GPU kernels / copies. */
dt_status dt_pack_host(dt_t t, int64_t count, const void* origin, void* packed, int64_t pos, int64_t* len,
                       void* stream);
dt_status dt_unpack_host(dt_t t, int64_t count, const void* packed, void* origin, int64_t pos, int64_t* len,
                         void* stream);

/* Fused datatype -> datatype copy on the current device:
 * dst' = unpack(rtype, rcount, pack(stype, scount, src)) over the first
 * scount*size(stype) bytes, without a packed intermediate: every stream byte
 * goes from its source-layout address (src, D) straight to its
 * destination-layout address (dst, D).  Signatures may differ (reading A12;
 * vector <-> contiguous, matrix transpose: [L26:c4303 §5.2.2], [L26:c4896
 * §5.2.3]); a larger receive fills a prefix.  Errors: DT_ERR_TRUNCATE if the
 * bytes do not fit, DT_ERR_OVERLAP for an overlapping destination typemap,
 * DT_ERR_NOT_COMMITTED, DT_ERR_ARG.  Asynchronous on `stream`. */
dt_status dt_copy(dt_t stype, int64_t scount, const void* src, dt_t rtype, int64_t rcount, void* dst, void* stream);

/* ------------------------------------------------------------------ introspection (host only, no GPU) */
typedef struct {
  int64_t size, lb, extent, true_lb, true_extent;
  int64_t nblocks;        /* blocks in the template (one element), after merging */
  int64_t tsize;          /* bytes per template element                            */
  int32_t nlevels;        /* strided / list levels above the template (outermost first) */
  int32_t level_is_list[8];
  int64_t level_count[8];
  int64_t level_stride[8];/* bytes; 0 for list levels                             */
  int64_t granularity;    /* largest power of two <= 16 dividing every disp/len/stride */
} dt_form_info;
/* Builds (and caches) the flattened host form without touching the GPU. */
dt_status dt_get_form(dt_t t, dt_form_info* out);
/* Expand `count` instances into merged (disp, len) blocks in typemap order
 * (host arrays of capacity max); *nblocks = total blocks (may exceed max). */
dt_status dt_flatten(dt_t t, int64_t count, int64_t* disps, int64_t* lens, int64_t max, int64_t* nblocks);
/* Which kernel dt_pack would launch for this request: 0 none, 1 warp-segment
 * ("long"), 2 word-table ("short", register staged), 3 block windows (short
 * blocks under a large template), 4 shared-memory/TMA staging, 6 record spans
 * (short blocks inside small dense records); *granularity = word size in bytes. */
dt_status dt_plan(dt_t t, int64_t count, uint64_t origin_addr, uint64_t packed_addr, int64_t pos, int64_t len,
                  int* kernel, int64_t* granularity);

/* Ship a layout to another rank: the flattened form (levels + block template +
 * index tables, native byte order: homogeneous GPUs, reading A5) and the bounds.
 * dt_type_serialize: out == NULL -> *nbytes = required size; else writes up to
 * *nbytes (DT_ERR_ARG if too small).  dt_type_deserialize: a new uncommitted
 * handle (one reference) whose typemap equals the serialized type's; it has no
 * constructor tree but can be committed, packed and used as a component.
 * Host only.  Errors: DT_ERR_ARG (NULL, malformed blob), DT_ERR_NOMEM. */
dt_status dt_type_serialize(dt_t t, void* out, size_t* nbytes);
dt_status dt_type_deserialize(const void* in, size_t nbytes, dt_t* out);

/* ------------------------------------------------------------------ GPU <-> GPU transfer */
enum { DT_XFER_P2P = 0, DT_XFER_NCCL = 1, DT_XFER_CE = 2 };
typedef struct {
  int64_t chunk_bytes; /* pipeline fragment size C (reading A15); 0 = default 1 MiB; <= 1 GiB */
  int32_t depth;       /* ring slots D (fragments in flight) per (peer, channel), <= 256;
                          0 = auto: D*C >= 8 MiB, at least 4 slots (NCCL mode: 4)      */
  int32_t mode;        /* DT_XFER_P2P (pack straight into the peer's ring over NVLink),
                          DT_XFER_NCCL (double-buffered ncclSend/ncclRecv of packed chunks) or
                          DT_XFER_CE (pack into local staging, copy-engine copy into the peer's
                          ring, stream-ordered flag kernels; host-driven, a comparator) */
  int32_t ctas;        /* CTAs per direction for the P2P pipeline kernel; 0 = default      */
  int32_t flags;       /* bit 0: loopback (dest = source = self) through the ring pipeline
                          instead of the fused datatype -> datatype copy (dt_copy)        */
} dt_xfer_opts;

/* Create this rank's endpoint on `device`: allocates the receive rings
 * (nranks*6 channels*depth*chunk bytes) and flag words, and (mode NCCL)
 * initialises a NCCL communicator from `nccl_unique_id` (128 B, H; may be NULL
 * for P2P).  Every rank must use the same chunk_bytes, depth and mode
 * (dt_comm_connect checks; DT_ERR_ARG otherwise).  The handle is single-threaded
 * and its operations must be stream-ordered (one stream, or joined streams): a
 * receive posts "start packing" when its kernel starts, which tells the sender
 * that the previous message on the channel has been consumed. */
dt_status dt_comm_init(int rank, int nranks, const void* nccl_unique_id, int device, const dt_xfer_opts* o,
                       dt_comm_t* out);
/* NCCL unique id for rank 0 to broadcast (H buffer of 128 bytes). */
dt_status dt_nccl_unique_id(void* out128);
/* This rank's IPC handles (rings + flags); *nbytes in: capacity, out: used. */
dt_status dt_comm_local_handle(dt_comm_t c, void* out, size_t* nbytes);
/* After the caller all-gathered every rank's handle blob (H, nranks *
 * nbytes_per_rank, rank-major): map every peer's ring/flags once
 * (cudaIpcOpenMemHandle; [L20:c3807 §4.1]).  Same-process peers (loopback) are
 * recognised and not re-mapped.  DT_ERR_ARG if a peer's chunk/depth/mode differ. */
dt_status dt_comm_connect(dt_comm_t c, const void* all_handles, size_t nbytes_per_rank);
/* Send scount instances of stype from sbuf (D) to rank `dest` and receive into
 * rbuf (D) rcount instances of rtype from rank `source` (either may be -1 =
 * none; dest/source may equal this rank = loopback, the paper's "1GPU" case
 * [L26:c1686]).  Signatures may differ as long as the byte counts fit
 * (reading A12): the receive fills a prefix; scount*size(stype) >
 * rcount*size(rtype) of the matching peer is DT_ERR_TRUNCATE, detected before
 * any byte moves (the receiver posts its capacity with "start packing"
 * [L20:c3973], the sender compares before its first fragment).
 * Pipelined in fragments of chunk_bytes through `depth` ring slots: cost ~
 * transfer + one fragment's pack/unpack ([L18:c4932 §4.1]).  Enqueued on
 * `stream`; returns without host synchronisation (P2P mode). */
dt_status dt_sendrecv(const void* sbuf, int64_t scount, dt_t stype, int dest, void* rbuf, int64_t rcount, dt_t rtype,
                      int source, dt_comm_t c, const dt_xfer_opts* o, void* stream);
/* Batch several sendrecv calls (halo: 6 faces to 3 peers) and issue them
 * together, deadlock-free. */
dt_status dt_group_start(dt_comm_t c);
dt_status dt_group_end(dt_comm_t c, void* stream);
/* Poll/return the sticky device-side error flag (timeouts, truncation). */
dt_status dt_comm_check(dt_comm_t c);
dt_status dt_comm_free(dt_comm_t* c);

/* ------------------------------------------------------------------ persistent direct exchange
 * SURVEY §8(f) f1 across GPUs: the datatype -> datatype copy of dt_copy, with
 * the destination in the PEER's memory.  A plan is a fixed set of sends and
 * receives (an MPI persistent request set: the C4 halo's 6 + 6 faces); once
 * connected, every dt_xplan_start is ONE kernel per rank that
 *   1. posts this rank's receive buffers (release-stores "ready" = seq into each
 *      source's flag page over NVLink),
 *   2. copies every send straight from the local layout into the receiver's
 *      layout in peer HBM (the receiver's flattened type was shipped at connect;
 *      no ring, no packed intermediate, no receiver-side unpack: each byte is
 *      read once and written once), after the receiver posted it,
 *   3. publishes "done" = seq to each receiver (system-scope fence first) and
 *      waits until all of this rank's receives are done,
 * so the stream order after dt_xplan_start sees the received data.  The paper's
 * pipeline exists to overlap pack / transfer / unpack ([L18:c4932 §4.1]); here
 * all three are one pass over NVLink peer memory.
 * Matching: send (dest d, tag t) of rank r <-> receive (source r, tag t) of d.
 * Truncation (send bytes > receive capacity) is DT_ERR_TRUNCATE at connect,
 * before any byte moves; an overlapping receive typemap is DT_ERR_OVERLAP.
 * Every rank must start its plan the same number of times (collective);
 * waits are bounded (DT_TIMEOUT_MS) and reported by dt_xplan_check. */
typedef struct dt_xplan_s* dt_xplan_t;
typedef struct {
  void* buf;      /* D: origin of the layout (send: read; receive: written)          */
  int64_t count;  /* instances of type                                              */
  dt_t type;      /* committed type                                                 */
  int32_t peer;   /* destination (send) / source (receive) rank; may be this rank   */
  int32_t tag;    /* matching key of a (sender, receiver) pair                       */
} dt_xop;
/* Local part (allocates the flag page on the comm's device). nsend, nrecv <= 16. */
dt_status dt_xplan_create(dt_comm_t c, int nsend, const dt_xop* sends, int nrecv, const dt_xop* recvs,
                          dt_xplan_t* out);
/* What this rank exports to its peers (IPC handles of the receive buffers and of
 * the flag page, serialized receive types); out == NULL -> *nbytes = size. */
dt_status dt_xplan_local_blob(dt_xplan_t p, void* out, size_t* nbytes);
/* blobs: every rank's blob concatenated in rank order (H), sizes[r] bytes each.
 * Maps peers' buffers once (cudaIpcOpenMemHandle, cached per comm), commits the
 * receivers' types on this device and builds the launch. */
dt_status dt_xplan_connect(dt_xplan_t p, const void* blobs, const size_t* sizes);
dt_status dt_xplan_start(dt_xplan_t p, void* stream);
dt_status dt_xplan_check(dt_xplan_t p);  /* sticky device-side error (timeout) */
dt_status dt_xplan_free(dt_xplan_t* p);

const char* dt_last_error(void);
const char* dt_version(void);

#ifdef __cplusplus
}
#endif
#endif
