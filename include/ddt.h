/*
 * ddt.h -- C ABI of the B200-native dynamic-kernel-fusion library for bulk
 * non-contiguous (MPI derived datatype) pack / unpack and halo exchange.
 *
 * Paper: Chu, Khorassani, Zhou, Subramoni, Panda, "Dynamic Kernel Fusion for
 * Bulk Non-contiguous Data Transfer on GPU Clusters" (/root/reference/PAPER.md,
 * cited as P:<line>).  The calls follow the paper's problem statement:
 *   - datatype construction + commit            Alg 1/3 lines 1-2
 *   - cached data layout entry                  §IV-A.1, §IV-B.1
 *   - request list (circular, Head/Tail, UID)   §IV-A.1
 *   - scheduler (1) enqueue  (2) one fused launch (3) GPU completion (4) query
 *                                               §IV-A.2
 *   - negative UID => caller falls back
 *   - fused kernel over an array of requests    §IV-A.3
 *   - halo exchange, one message per boundary buffer   Alg 3, §IV-B
 * Datatype semantics are MPI-3.1 §4.1 (the paper defers to the standard, ref [29]).
 *
 * Conventions (all entry points):
 *   - Every function returns a ddt_status_t (0 = DDT_OK, < 0 = error) or, for
 *     enqueue, a uid >= 0 / error < 0.  Nothing aborts, exits or throws across
 *     the ABI.  CUDA / NCCL failures are sticky on the queue and reported by
 *     the next call on it (DDT_ERR_CUDA / DDT_ERR_NCCL); ddt_strerror() and
 *     ddt_last_error_message() describe them.
 *   - Ownership: the library owns type objects, device layout caches, request
 *     rings, descriptor tables, staging buffers, windows it allocates and halo
 *     plans.  The CALLER owns every data buffer and must keep it alive and
 *     unmodified until the request is COMPLETED (MPI non-blocking semantics,
 *     P:241).  A data buffer is device memory of the queue's device, a
 *     peer-mapped device pointer, or PAGE-LOCKED HOST memory (cudaHostAlloc /
 *     cudaHostRegister; unified addressing): the fused kernel then reads /
 *     writes exactly the typemap's bytes over PCIe with no staging copy (the
 *     zero-copy path; tests/test_gpu_hostmem.py).  Pageable host memory is not
 *     accepted (the kernel would fault).  P2P / P2P_DIRECT halo plans need
 *     device memory for the buffers they open through CUDA IPC.
 *   - Byte displacements are signed 64-bit and relative to the user pointer;
 *     the caller guarantees the whole footprint is inside its allocation
 *     (reading R4).
 *   - Packed format: exactly count*size bytes, entries in typemap order, no
 *     header, no padding (R1, R8).  Instance k of a count sits at k*extent (R9).
 *   - Threads: committed types are immutable and may be shared across threads;
 *     a queue / halo belongs to one host thread.
 */
#ifndef DDT_H
#define DDT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t ddt_status_t;

enum {
    DDT_OK = 0,
    DDT_ERR_ARG = -1,           /* invalid argument (bad sizes, NULL, count < 0, ...) */
    DDT_ERR_STATE = -2,         /* type not committed, freed handle, bad lifecycle */
    DDT_ERR_QUEUE_FULL = -3,    /* request ring full: the paper's negative UID; flush and retry */
    DDT_ERR_OVERLAP = -4,       /* unpack into a typemap with overlapping entries (R5) */
    DDT_ERR_NOMEM = -5,         /* host or device allocation failed */
    DDT_ERR_CUDA = -6,          /* a CUDA runtime call failed (sticky on the queue) */
    DDT_ERR_NCCL = -7,          /* an NCCL call failed */
    DDT_ERR_SIZE_MISMATCH = -8, /* matched send/recv pair with different packed sizes */
    DDT_ERR_TIMEOUT = -9,       /* a device-side wait for a peer flag exceeded its bound */
    DDT_ERR_UNSUPPORTED = -10,  /* feature not built / too large for the device descriptor */
    DDT_ERR_NODEV = -11         /* no CUDA device visible */
};

/* Basic (predefined) types; size = alignment = 1, 4, 8, 4, 8 bytes. */
enum ddt_base { DDT_BYTE = 0, DDT_INT32 = 1, DDT_INT64 = 2, DDT_FLOAT = 3, DDT_DOUBLE = 4 };
enum ddt_order { DDT_ORDER_C = 0, DDT_ORDER_FORTRAN = 1 };
/* Request / response status values. */
enum ddt_state { DDT_IDLE = 0, DDT_PENDING = 1, DDT_BUSY = 2, DDT_COMPLETED = 3 };
/* Flattened layout kinds of the layout cache (R7). */
enum ddt_layout_kind { DDT_LAYOUT_EMPTY = 0, DDT_LAYOUT_STRIDED = 1, DDT_LAYOUT_UNIFORM_LIST = 2,
                       DDT_LAYOUT_GENERAL_LIST = 3 };
/* Exchange modes. */
enum ddt_xchg_mode {
    DDT_XCHG_NCCL = 0,  /* fused pack -> grouped ncclSend/ncclRecv per peer -> fused unpack */
    DDT_XCHG_P2P = 1,   /* ONE kernel: pack straight into peers' windows over NVLink,
                           release a per-message flag, unpack each message on arrival */
    DDT_XCHG_P2P_DIRECT = 2, /* ONE kernel, pack-free (DirectIPC): gather the
                           send layout and scatter straight into the peer's receive layout
                           through a CUDA-IPC mapping of its buffer, after the peer's
                           "ready" flag; needs closed-form (strided) receive types */
    DDT_XCHG_NCCL_EARLY = 3  /* NCCL mode with per-peer early send (the sender
                           sends "as soon as any packing request is completed"): the
                           fused pack kernel counts each message's completion in device
                           memory (the CTA finishing its last item), and each remote
                           peer's ncclSend/ncclRecv group waits on its own stream
                           (stream memory operation on those counters) for that peer's
                           messages only, not for the whole pack batch */
};

typedef struct ddt_type_s* ddt_type_t;   /* opaque, library-owned, immutable after commit */
typedef struct ddt_queue_s* ddt_queue_t; /* bound to (device, cudaStream_t); one host thread */
typedef struct ddt_halo_s* ddt_halo_t;   /* a persistent exchange plan */

/* ------------------------------------------------------------------ types
 * MPI-3.1 §4.1 constructors ("vector, indexed, subarray, struct, and
 * more").  `old` may be a basic or any derived type (nesting, D2 in SURVEY).
 * Counts / block lengths must be >= 0; zero-length blocks and count 0 give
 * entries-free types (R3).  Strides / displacements may be negative (R4).
 * The new type holds a reference on `old`; ddt_free(old) afterwards is safe.
 * Errors: DDT_ERR_ARG for invalid parameters, DDT_ERR_NOMEM.               */
ddt_status_t ddt_type_basic(int base, ddt_type_t* out);      /* predefined; freeing it is a no-op */
ddt_status_t ddt_create_contiguous(int64_t count, ddt_type_t old, ddt_type_t* out);
/* vector: count blocks of blocklen old elements, block starts `stride` OLD EXTENTS apart */
ddt_status_t ddt_create_vector(int64_t count, int64_t blocklen, int64_t stride, ddt_type_t old,
                               ddt_type_t* out);
/* hvector: as vector with the stride in BYTES */
ddt_status_t ddt_create_hvector(int64_t count, int64_t blocklen, int64_t stride_bytes, ddt_type_t old,
                                ddt_type_t* out);
/* indexed: block i = blocklens[i] old elements at displs[i] OLD EXTENTS (arrays are copied) */
ddt_status_t ddt_create_indexed(int64_t count, const int64_t* blocklens, const int64_t* displs,
                                ddt_type_t old, ddt_type_t* out);
/* hindexed: as indexed with displacements in BYTES (need not be multiples of the element size, R20) */
ddt_status_t ddt_create_hindexed(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes,
                                 ddt_type_t old, ddt_type_t* out);
/* indexed_block / hindexed_block: every block has `blocklen` elements (MPI-3.1 §4.1.2) */
ddt_status_t ddt_create_indexed_block(int64_t count, int64_t blocklen, const int64_t* displs, ddt_type_t old,
                                      ddt_type_t* out);
ddt_status_t ddt_create_hindexed_block(int64_t count, int64_t blocklen, const int64_t* displs_bytes, ddt_type_t old,
                                       ddt_type_t* out);
/* struct: block i = blocklens[i] copies of types[i] at byte displacement
 * displs_bytes[i] (+ j * extent(types[i])).  Heterogeneous blocks (e.g. the
 * paper's struct-on-indexed specfem3D_cm layout).  The upper bound carries
 * MPI's alignment increment epsilon (MPI-3.1 §4.1; reading R2): the extent is
 * rounded up to a multiple of the largest basic-type alignment (= its size) in
 * the typemap, e.g. {(double,0),(byte,8)} has extent 16 -- unless a block's
 * type has explicit bounds (resized / subarray beneath it), which then rule. */
ddt_status_t ddt_create_struct(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes,
                               const ddt_type_t* types, ddt_type_t* out);
/* resized (MPI-3.1 §4.1.7): the typemap of `old` with lb / extent replaced;
 * instances of a count and copies inside parent types step by `extent`.
 * extent >= 0.  A type without entries still contributes no bounds (R3). */
ddt_status_t ddt_create_resized(ddt_type_t old, int64_t lb, int64_t extent, ddt_type_t* out);
/* subarray (MPI-3.1 §4.1.3): 1 <= ndims <= 16, 1 <= subsizes[k] <= sizes[k],
 * 0 <= starts[k] <= sizes[k]-subsizes[k]; result has lb 0 and extent prod(sizes)*ext(old). */
ddt_status_t ddt_create_subarray(int ndims, const int64_t* sizes, const int64_t* subsizes,
                                 const int64_t* starts, int order, ddt_type_t old, ddt_type_t* out);

/* Commit = flatten the typemap into the layout cache: segments
 * in typemap order, adjacent-merged, classified STRIDED (closed-form <= 4 dims,
 * zero metadata), UNIFORM_LIST (one length, 32/64-bit offsets) or GENERAL_LIST
 * (offset, length, packed prefix); size / lb / extent / true extent / overlap
 * flag are recorded.  The device copy of the cache is uploaded once per device
 * on first use by a queue of that device (host-only commit works without a GPU).
 * Idempotent.  Errors: DDT_ERR_ARG (NULL), DDT_ERR_NOMEM.                     */
ddt_status_t ddt_commit(ddt_type_t t);
/* Drops the caller's reference; deferred while in-flight requests reference
 * the type.  Sets *t = NULL.  Freeing a basic type is a no-op.               */
ddt_status_t ddt_free(ddt_type_t* t);

/* Closed-form queries (valid before commit). */
ddt_status_t ddt_get_size(ddt_type_t t, int64_t* size);
ddt_status_t ddt_get_extent(ddt_type_t t, int64_t* lb, int64_t* extent);
ddt_status_t ddt_get_true_extent(ddt_type_t t, int64_t* true_lb, int64_t* true_extent);
/* Introspection of the committed layout (DDT_ERR_STATE before commit). */
ddt_status_t ddt_get_num_segments(ddt_type_t t, int64_t* nseg);
ddt_status_t ddt_get_layout_kind(ddt_type_t t, int32_t* kind);
/* Copies up to `cap` segments (byte offset, byte length) of ONE instance in
 * typemap (= packed) order; *n receives the total number of segments. */
ddt_status_t ddt_get_segments(ddt_type_t t, int64_t* offsets, int64_t* lengths, int64_t cap, int64_t* n);
/* 1 if two entries of one instance overlap (unpack is then rejected, R5). */
ddt_status_t ddt_get_overlaps(ddt_type_t t, int32_t* overlaps);

/* ------------------------------------------------------------------ queue
 * A queue = the paper's request list + scheduler bound to one
 * device and one CUDA stream (cudaStream_t passed as void*, NULL = legacy
 * default stream).  capacity = ring size (0 => 4096, R11).  Every launch
 * made through a queue (flushes, its plans, its halo plans) goes to that
 * stream; when such launches are captured into CUDA graphs, replays must stay
 * ordered with each other (large batches share the queue's work-ticket
 * counter, device_desc.h).
 * Errors: DDT_ERR_NODEV, DDT_ERR_CUDA, DDT_ERR_NOMEM, DDT_ERR_ARG.          */
ddt_status_t ddt_queue_create(int device, void* cuda_stream, int32_t capacity, ddt_queue_t* out);
/* Waits for in-flight work, then frees the queue. */
ddt_status_t ddt_queue_destroy(ddt_queue_t q);

/* Scheduler (1): append a request at Tail and return its uid >= 0 (R12), or
 * a negative error: DDT_ERR_QUEUE_FULL (ring full), DDT_ERR_STATE
 * (type not committed), DDT_ERR_ARG (count < 0, NULL buffer with size > 0,
 * request of >= 2^32 vectors), DDT_ERR_OVERLAP (unpack into an overlapping
 * type).  Nothing runs until ddt_flush.  A zero-byte request is COMPLETED at
 * once.
 *   pack:   src = non-contiguous device buffer (MPI buffer address),
 *           dst_packed = contiguous device buffer of count*size bytes.
 *   unpack: src_packed = contiguous device buffer of count*size bytes,
 *           dst = non-contiguous device buffer.
 * Requests flushed together must not alias: write sets pairwise disjoint and
 * disjoint from every read set (R6); the result is then order-independent. */
int64_t ddt_pack_enqueue(ddt_queue_t q, ddt_type_t t, const void* src, int64_t count, void* dst_packed);
int64_t ddt_unpack_enqueue(ddt_queue_t q, ddt_type_t t, const void* src_packed, int64_t count, void* dst);

/* Bulk enqueue: n requests of one operation in one call (the loop of
 * Alg 3 lines 3-6, without a per-request trip across the ABI --
 * the per-call cost of a binding such as ctypes dwarfs the ~0.1 us enqueue).
 *   op      DDT_OP_PACK (0) or DDT_OP_UNPACK (1);
 *   types   [n] committed types;  srcs / dsts [n] buffers as for
 *           ddt_pack_enqueue / ddt_unpack_enqueue;  counts [n];
 *   uids_out [n] (may be NULL) receives each request's uid.
 * Requests are appended in array order.  Returns k = the number enqueued
 * (n on success); if k < n, request k failed with the negative status
 * returned in uids_out[k] (if given) and requests k..n-1 were not enqueued
 * -- on DDT_ERR_QUEUE_FULL the caller flushes and resubmits from k.
 * A negative return (DDT_ERR_ARG) means nothing was enqueued.               */
enum { DDT_OP_PACK = 0, DDT_OP_UNPACK = 1 };
int64_t ddt_enqueue_many(ddt_queue_t q, int32_t op, int64_t n, const ddt_type_t* types, const void* const* srcs,
                         const int64_t* counts, void* const* dsts, int64_t* uids_out);

/* DirectIPC request ("a direct non-contiguous data transfer", fused with
 * packing / unpacking in one kernel): gather `src_count` instances of
 * `src_type` at `src` and scatter them as `dst_count` instances of `dst_type`
 * at `dst`, with no packed intermediate.  The packed sizes must match
 * (DDT_ERR_SIZE_MISMATCH) and dst_type must not overlap (DDT_ERR_OVERLAP).
 * Both pointers are device pointers of the queue's device (or peer-mapped).
 * Returns a uid >= 0 or a negative error, like the other enqueues.          */
int64_t ddt_direct_enqueue(ddt_queue_t q, ddt_type_t src_type, const void* src, int64_t src_count,
                           ddt_type_t dst_type, void* dst, int64_t dst_count);

/* Scheduler (2): launch every pending request (Head..Tail) as ONE fused
 * kernel on the queue's stream (P:217, P:221, P:255 trigger (1)).  Returns
 * the number of requests launched (0 => nothing pending, no launch) or < 0.
 * DDT_ERR_STATE while the queue's stream is being captured into a CUDA graph
 * (the requests stay pending): graphs capture ddt_plan_launch / ddt_exchange. */
int32_t ddt_flush(ddt_queue_t q);
/* Scheduler (4): state of a uid: *state = DDT_PENDING (enqueued, not
 * flushed), DDT_BUSY (flushed, GPU not done), DDT_COMPLETED.  Non-blocking.
 * DDT_ERR_ARG for an unknown / future uid.                                   */
ddt_status_t ddt_query(ddt_queue_t q, int64_t uid, int32_t* state);
/* Host-blocks until every flushed batch of the queue is complete.  Pending
 * (unflushed) requests are flushed first (MPI_Waitall semantics).    */
ddt_status_t ddt_wait(ddt_queue_t q);

/* Persistent batch (static-batch replay; SURVEY §8(d) config 5 "fused + graph
 * replay" arm): moves every pending request of q into a plan whose device work
 * table is uploaded once.  The moved uids complete in q's request list at once
 * (they are never launched by ddt_flush); each ddt_plan_launch is ONE fused
 * launch of the whole batch on q's stream.  The caller's buffers must stay
 * valid for the plan's lifetime.  Errors: DDT_ERR_ARG, DDT_ERR_CUDA, DDT_ERR_NOMEM. */
typedef struct ddt_plan_s* ddt_plan_t;
ddt_status_t ddt_plan_create(ddt_queue_t q, ddt_plan_t* out);
ddt_status_t ddt_plan_launch(ddt_plan_t p);
ddt_status_t ddt_plan_destroy(ddt_plan_t p);

/* Scheduler trigger (2) of §IV-C: once the pending requests hold
 * >= `bytes` packed bytes, the enqueue that crossed the threshold also flushes
 * (the paper's fusion threshold; ~512 KB on V100, to be re-tuned on B200).
 * 0 (the default) = launch only on explicit ddt_flush / ddt_wait (trigger (1),
 * the synchronisation point).  Errors: DDT_ERR_ARG. */
ddt_status_t ddt_queue_set_flush_threshold(ddt_queue_t q, int64_t bytes);
/* Scheduler (3) per request: when enabled, the GPU thread that
 * finishes a request's last work item writes its response status into
 * host-mapped memory, so ddt_query reports DDT_COMPLETED for that request as
 * soon as it is done -- before the rest of its fused batch -- without any host
 * synchronisation.  Default off (batch-level completion by CUDA event; the
 * per-item bookkeeping costs one atomic per work item).  Only between batches
 * (DDT_ERR_STATE if requests are pending). */
ddt_status_t ddt_queue_set_response_flags(ddt_queue_t q, int32_t enable);

/* Counters since queue creation: requests enqueued, fused kernel launches,
 * flushes, packed bytes moved (pack + unpack), and requests that moved as
 * phased 16-B units (closed-form rows at 8 mod 16 on both sides, DESIGN.md
 * "phased units"; introspection only).                                      */
typedef struct {
    int64_t requests, launches, flushes, bytes, phased;
} ddt_queue_stats_t;
ddt_status_t ddt_queue_get_stats(ddt_queue_t q, ddt_queue_stats_t* out);

/* ------------------------------------------------------------------ halo
 * A persistent halo-exchange plan (Alg 3: one Isend + one Irecv per boundary
 * buffer).  A send to (peer, tag) matches the peer's receive from
 * (this rank, tag); (peer, tag) pairs are unique per direction (R16).       */
typedef struct {
    int32_t peer, tag;
    ddt_type_t type;   /* committed */
    const void* buf;   /* non-contiguous device source (send) */
    int64_t count;
} ddt_send_t;
typedef struct {
    int32_t peer, tag;
    ddt_type_t type;   /* committed, non-overlapping */
    void* buf;         /* non-contiguous device destination (recv) */
    int64_t count;
} ddt_recv_t;

/* Communication context.  nranks == 1 needs neither NCCL nor windows (every
 * message is a self message).  The one-time plan metadata exchange (directory
 * of tags / sizes / window offsets, and an agreed status) uses host_allgather
 * when given -- any process group, e.g. torch.distributed over gloo or NCCL --
 * else NCCL.  DDT_XCHG_NCCL needs nccl_comm (an ncclComm_t from
 * ddt_nccl_comm_create) for its data path.  DDT_XCHG_P2P needs peer_windows
 * [nranks] (device pointers, valid on this device, to every rank's window --
 * this rank's own included -- each >= ddt_halo_window_bytes() bytes).
 * host_allgather(ctx, send, bytes, recv) must gather `bytes` bytes from every
 * rank into recv[nranks * bytes] in rank order and return 0 (collective). */
typedef int32_t (*ddt_allgather_fn)(void* ctx, const void* send, int64_t bytes, void* recv);
typedef struct {
    int32_t rank, nranks;
    void* nccl_comm;
    void* const* peer_windows;
    int64_t window_bytes;
    ddt_allgather_fn host_allgather;
    void* host_ctx;
} ddt_comm_t;

/* Bytes of window a rank needs for DDT_XCHG_P2P with the given receives. */
ddt_status_t ddt_halo_window_bytes(int32_t nrecv, const ddt_recv_t* recvs, int64_t* bytes);
/* Build the plan: validates, matches sizes with the peers (one metadata
 * exchange when nranks > 1), allocates staging, builds the device work tables
 * once.  Collective over all ranks of the comm.
 * Errors: DDT_ERR_ARG, DDT_ERR_STATE, DDT_ERR_SIZE_MISMATCH, DDT_ERR_NCCL,
 * DDT_ERR_CUDA, DDT_ERR_NOMEM, DDT_ERR_OVERLAP.                              */
ddt_status_t ddt_halo_create(ddt_queue_t q, const ddt_comm_t* comm, int32_t nsend, const ddt_send_t* sends,
                             int32_t nrecv, const ddt_recv_t* recvs, int32_t mode, ddt_halo_t* out);
/* One exchange iteration, asynchronous on the queue's stream: every send
 * packed, transferred, every receive unpacked.  NCCL mode: fused
 * pack launch -> grouped send/recv -> fused unpack launch (NCCL_EARLY: one
 * send/recv group per remote peer on its own stream, each started when that
 * peer's messages are packed, joined before the unpack).  P2P modes: a single
 * launch whose exchange epoch lives on the device, so every plan can be
 * captured into a CUDA graph by the caller (a K-step time loop) or replay its
 * own graph (ddt_halo_set_graph(h, 1)).  All ranks must issue the same
 * sequence of ddt_exchange calls.                                            */
ddt_status_t ddt_exchange(ddt_halo_t h);
ddt_status_t ddt_halo_set_graph(ddt_halo_t h, int32_t use_graph);
/* Bound of every device-side flag wait of a P2P plan (default 10 s).  A wait
 * that exceeds it abandons the message, sets a host-mapped error flag and
 * the next ddt_exchange returns DDT_ERR_TIMEOUT (sticky) -- never a hang.
 * Takes effect for launches issued afterwards (a captured graph is rebuilt). */
ddt_status_t ddt_halo_set_timeout(ddt_halo_t h, int64_t timeout_ns);
/* Tracing: record one 48-byte record per work item of the fused
 * P2P exchange kernel -- {u32 cta, item, request, op; u64 t_start, t_after_wait,
 * t_after_data, t_after_signal} in %globaltimer ns -- into dev_records (device
 * memory, `capacity` records; later records are dropped).  capacity 0 turns it
 * off.  Resets the record counter.  DDT_ERR_STATE for NCCL-mode plans. */
ddt_status_t ddt_halo_set_trace(ddt_halo_t h, void* dev_records, int64_t capacity);
/* Kernel launches issued by the last ddt_exchange (graph replay counts the
 * kernels inside the graph). */
ddt_status_t ddt_halo_launches_per_exchange(ddt_halo_t h, int32_t* launches);
/* Waits for the halo's queue, then frees the plan (not the caller's buffers). */
ddt_status_t ddt_halo_destroy(ddt_halo_t h);

/* ------------------------------------------------------------- NCCL / IPC
 * Plumbing for multi-process runs (one process per GPU): the Python layer
 * broadcasts the unique id / IPC handles through torch.distributed.         */
ddt_status_t ddt_nccl_unique_id(void* id_out /* 128 bytes */);
ddt_status_t ddt_nccl_comm_create(int32_t nranks, const void* id /* 128 bytes */, int32_t rank, void** comm_out);
ddt_status_t ddt_nccl_comm_destroy(void* comm);
/* Device window allocation for DDT_XCHG_P2P (zero-filled) + CUDA IPC. */
ddt_status_t ddt_window_alloc(int device, int64_t bytes, void** ptr_out, void* ipc_handle_out /* 64 bytes */);
ddt_status_t ddt_window_open(int device, const void* ipc_handle /* 64 bytes */, void** ptr_out);
ddt_status_t ddt_window_close(void* peer_ptr);
ddt_status_t ddt_window_free(void* ptr);

/* ------------------------------------------------------------------ misc */
const char* ddt_strerror(ddt_status_t s);
/* Thread-local text of the last error (CUDA / NCCL detail), "" if none. */
const char* ddt_last_error_message(void);
/* Experiment / test knobs (DDT_* environment variables, documented where they
 * are read) are read once and cached -- getenv costs ~0.1-0.3 us per call on
 * the flush path.  ddt_reload_env() makes the next use of every knob re-read
 * the environment (tests and A/B tools call it after changing a variable). */
void ddt_reload_env(void);
/* Library version and the SM architecture the kernels were built for (100). */
int32_t ddt_version(void);
int32_t ddt_built_sm(void);

#ifdef __cplusplus
}
#endif
#endif /* DDT_H */
