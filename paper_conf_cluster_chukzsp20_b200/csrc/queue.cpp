// queue.cpp -- the request list and scheduler of the kernel-fusion framework.
//
// Paper §IV-A:
//   * request list: a circular buffer with Head and Tail; each request has a
//     UID, an operation (Packing / Unpacking), origin / target buffers, the
//     cached data layout entry, a request status and a response status
//     (P:189-199).
//   * scheduler (1) enqueue at Tail and return the UID, negative when the list
//     is full so the caller can fall back; (2) launch ONE fused
//     kernel with an array of requests; (3) the GPU completes requests
//     without a host synchronisation at the kernel boundary; (4)
//     status query by UID comparing request and response status.
//   * a single host thread acts as scheduler.
// B200 realisation: the ring holds host request records;
// every request's device descriptor is built at enqueue (O(1)); ddt_flush
// turns [flushed, Tail) into a work table (item prefix sum) and issues ONE
// launch -- batches of <= 32 requests ride in the kernel parameters (one stream
// operation in total), larger ones are copied with one cudaMemcpyAsync first;
// completion of a batch is a CUDA event recorded after the launch (response
// status, readings R13/R15); ring entries are recycled once their batch's event
// has fired.
#include <algorithm>
#include <cstring>
#include <deque>
#include <vector>

#include <cuda_runtime.h>

#include "ddt_internal.h"

#include <atomic>
#include <mutex>

using namespace ddt;

struct ddt_queue_s {
    struct Req {
        int64_t uid;
        int op;
        ddt_type_s* t;
        ddt_type_s* t2;  // DIRECT destination type (else nullptr)
        int64_t bytes;
        ReqDesc desc;    // source descriptor, built at enqueue (O(1)); flush only serializes
        ReqDesc aux;     // destination descriptor
    };
    struct Batch {
        int64_t first, end;  // uid range
        cudaEvent_t ev;
    };
    struct HostSlot {
        void* p = nullptr;
        size_t cap = 0;
        cudaEvent_t ev = nullptr;
        bool used = false;
    };
    int device = 0;
    cudaStream_t stream = nullptr;
    int32_t capacity = 4096;
    std::vector<Req> ring;
    int64_t head = 0, flushed = 0, tail = 0;  // uids: [head, flushed) in flight, [flushed, tail) pending
    std::deque<Batch> inflight;
    std::vector<cudaEvent_t> event_pool;
    std::vector<HostSlot> slots;
    int next_slot = 0;
    void* dev_table = nullptr;
    size_t dev_cap = 0;
    ddt_status_t sticky = DDT_OK;
    ddt_queue_stats_t stats{};
    int sm_count = 148;
    HostBatch scratch;
    Launchable launch;
    // §IV-C trigger (2): flush once the pending requests hold >= threshold bytes (0 = off)
    int64_t threshold = 0;
    int64_t pending_bytes = 0;
    // scheduler (3) per request: GPU-written response status (host-mapped) + item counters
    bool resp_on = false;
    uint32_t* resp_host = nullptr;
    uint32_t* resp_dev = nullptr;
    uint32_t* done_ctr = nullptr;
    uint32_t* ticket = nullptr;  // device u32[2]: dynamic item tickets of this queue's (stream-ordered) launches
};

namespace {

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

cudaEvent_t get_event(ddt_queue_s* q) {
    if (!q->event_pool.empty()) {
        cudaEvent_t e = q->event_pool.back();
        q->event_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    return e;
}

void release_req(ddt_queue_s::Req& r) {
    type_release(r.t);
    type_release(r.t2);
    r.t = r.t2 = nullptr;
}

// Batches of one queue run on one stream, so they complete in order: the
// newest completed batch implies every older one.  One cudaEventQuery costs
// ~1.4 us of host time, so completion is found with O(log n) queries (newest
// first, then binary search) instead of one query per in-flight batch.
void release_batches(ddt_queue_s* q, size_t n) {
    for (size_t i = 0; i < n; i++) {
        auto& b = q->inflight.front();
        for (int64_t u = b.first; u < b.end; u++) release_req(q->ring[(size_t)(u % q->capacity)]);
        q->head = b.end;
        q->event_pool.push_back(b.ev);
        q->inflight.pop_front();
    }
}

void reclaim(ddt_queue_s* q, bool block) {
    if (q->inflight.empty()) return;
    const size_t n = q->inflight.size();
    cudaError_t e = block ? cudaEventSynchronize(q->inflight.back().ev) : cudaEventQuery(q->inflight.back().ev);
    if (e != cudaErrorNotReady) {
        if (e != cudaSuccess && q->sticky == DDT_OK) q->sticky = cuda_fail("batch completion", e);
        release_batches(q, n);
        return;
    }
    size_t lo = 0, hi = n - 1;  // batches [0, lo) known complete; batch hi known pending
    while (lo < hi) {
        const size_t mid = (lo + hi) / 2;
        cudaError_t m = cudaEventQuery(q->inflight[mid].ev);
        if (m == cudaErrorNotReady) {
            hi = mid;
        } else {
            if (m != cudaSuccess && q->sticky == DDT_OK) q->sticky = cuda_fail("batch completion", m);
            lo = mid + 1;
        }
    }
    release_batches(q, lo);
}

// Scheduler (1): claim the Tail slot (or fail with the paper's negative UID).
int64_t claim(ddt_queue_s* q) {
    if (q->tail - q->head >= q->capacity) {
        DeviceGuard g(q->device);
        reclaim(q, false);
        if (q->tail - q->head >= q->capacity) return DDT_ERR_QUEUE_FULL;  // negative UID
    }
    return q->tail;
}

// Publish the Tail slot, whose desc/aux the caller has already written in place.
int64_t commit_slot(ddt_queue_s* q, int op, ddt_type_s* t, ddt_type_s* t2, int64_t bytes) {
    int64_t uid = q->tail++;
    auto& r = q->ring[(size_t)(uid % q->capacity)];
    r.uid = uid;
    r.op = op;
    r.t = t;
    r.t2 = t2;
    type_retain(t);
    type_retain(t2);
    r.bytes = bytes;
    r.desc.uid_lo = (uint32_t)uid;
    if (q->resp_on && bytes > 0) {
        size_t slot = (size_t)(uid % q->capacity);
        r.desc.resp = (uint64_t)(uintptr_t)(q->resp_dev + slot);
        r.desc.resp_val = (uint32_t)(uid + 1);
        r.desc.done_ctr = (uint64_t)(uintptr_t)(q->done_ctr + slot);
    }
    q->stats.requests++;
    q->pending_bytes += bytes;
    if (q->threshold > 0 && q->pending_bytes >= q->threshold) ddt_flush(q);  // errors are sticky
    return uid;
}

int64_t commit_req(ddt_queue_s* q, int op, ddt_type_s* t, ddt_type_s* t2, int64_t bytes, const ReqDesc& d,
                   const ReqDesc& a) {
    auto& r = q->ring[(size_t)(q->tail % q->capacity)];
    r.desc = d;
    r.aux = a;
    return commit_slot(q, op, t, t2, bytes);
}

int64_t enqueue(ddt_queue_s* q, int op, ddt_type_s* t, const void* src, int64_t count, void* dst) {
    if (!q || !t || count < 0) return DDT_ERR_ARG;
    if (q->sticky != DDT_OK) return q->sticky;
    if (!t->committed) return DDT_ERR_STATE;
    int64_t bytes = count * t->size;
    if (bytes > 0 && (!src || !dst)) return DDT_ERR_ARG;
    if (op == OP_UNPACK && bytes > 0 && instances_overlap(t, count)) return DDT_ERR_OVERLAP;
    int64_t c = claim(q);
    if (c < 0) return c;
    // build straight into the free Tail slot (it is only published by commit_slot)
    auto& r = q->ring[(size_t)(c % q->capacity)];
    if (bytes > 0) {
        DeviceLayout* dl = nullptr;
        ddt_status_t s = type_device_layout(t, q->device, &dl);
        if (s != DDT_OK) return s;
        s = build_request(op, t, dl, src, dst, count, &r.desc, &r.aux);
        if (s != DDT_OK) return s;
    } else {
        std::memset(&r.desc, 0, sizeof(r.desc));
        std::memset(&r.aux, 0, sizeof(r.aux));
    }
    return commit_slot(q, op, t, nullptr, bytes);
}

ddt_status_t ensure_host_slot(ddt_queue_s* q, size_t bytes, ddt_queue_s::HostSlot** out) {
    auto& s = q->slots[(size_t)q->next_slot];
    q->next_slot = (q->next_slot + 1) % (int)q->slots.size();
    if (s.used) {
        cudaError_t e = cudaEventSynchronize(s.ev);
        if (e != cudaSuccess) return cuda_fail("table slot", e);
    }
    if (s.cap < bytes) {
        if (s.p) cudaFreeHost(s.p);
        size_t cap = std::max<size_t>(bytes, 64 << 10);
        cudaError_t e = cudaHostAlloc(&s.p, cap, cudaHostAllocDefault);
        if (e != cudaSuccess) {
            s.p = nullptr;
            s.cap = 0;
            return cuda_fail("cudaHostAlloc(table)", e);
        }
        s.cap = cap;
    }
    if (!s.ev) cudaEventCreateWithFlags(&s.ev, cudaEventDisableTiming);
    *out = &s;
    return DDT_OK;
}

// Gather the pending requests' descriptors into q->scratch.
int64_t gather_pending(ddt_queue_s* q) {
    HostBatch& b = q->scratch;
    b.clear();
    int64_t moved = 0;
    for (int64_t u = q->flushed; u < q->tail; u++) {
        auto& r = q->ring[(size_t)(u % q->capacity)];
        if (r.bytes == 0) continue;
        b.add(r.desc, r.aux);
        moved += r.bytes;
    }
    phase_batch(b);
    if (q->resp_on) {  // the finishing CTA compares its count with the request's item count
        int ub = choose_ub(b, q->sm_count);
        for (auto& d : b.descs) d.nitems = desc_items(d, ub);
    }
    q->pending_bytes = 0;
    return moved;
}

}  // namespace

extern "C" {

ddt_status_t ddt_queue_create(int device, void* cuda_stream, int32_t capacity, ddt_queue_t* out) {
    if (!out || capacity < 0) return DDT_ERR_ARG;
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
        cudaGetLastError();
        ddt::set_error("no CUDA device visible");
        return DDT_ERR_NODEV;
    }
    if (device < 0 || device >= n) return DDT_ERR_ARG;
    auto* q = new (std::nothrow) ddt_queue_s();
    if (!q) return DDT_ERR_NOMEM;
    q->device = device;
    q->stream = (cudaStream_t)cuda_stream;
    q->capacity = capacity == 0 ? 4096 : capacity;
    q->ring.resize((size_t)q->capacity);
    q->slots.resize(4);
    {
        DeviceGuard g(device);
        cudaError_t e = cudaFree(nullptr);  // make the context current
        if (e != cudaSuccess) {
            delete q;
            return cuda_fail("context init", e);
        }
        q->sm_count = device_sm_count(device);
        e = cudaMalloc((void**)&q->ticket, 16);
        if (e == cudaSuccess) e = cudaMemset(q->ticket, 0, 16);
        if (e != cudaSuccess) {
            if (q->ticket) cudaFree(q->ticket);
            delete q;
            return cuda_fail("ticket counter", e);
        }
    }
    *out = q;
    return DDT_OK;
}

ddt_status_t ddt_queue_destroy(ddt_queue_t q) {
    if (!q) return DDT_ERR_ARG;
    {
        DeviceGuard g(q->device);
        reclaim(q, true);
        for (int64_t u = q->flushed; u < q->tail; u++) release_req(q->ring[(size_t)(u % q->capacity)]);
        for (auto e : q->event_pool) cudaEventDestroy(e);
        for (auto& s : q->slots) {
            if (s.p) cudaFreeHost(s.p);
            if (s.ev) cudaEventDestroy(s.ev);
        }
        if (q->dev_table) cudaFree(q->dev_table);
        if (q->resp_host) cudaFreeHost(q->resp_host);
        if (q->done_ctr) cudaFree(q->done_ctr);
        if (q->ticket) cudaFree(q->ticket);
    }
    delete q;
    return DDT_OK;
}

ddt_status_t ddt_queue_set_flush_threshold(ddt_queue_t q, int64_t bytes) {
    if (!q || bytes < 0) return DDT_ERR_ARG;
    q->threshold = bytes;
    if (bytes > 0 && q->pending_bytes >= bytes) {
        int32_t f = ddt_flush(q);
        if (f < 0) return f;
    }
    return DDT_OK;
}

ddt_status_t ddt_queue_set_response_flags(ddt_queue_t q, int32_t enable) {
    if (!q) return DDT_ERR_ARG;
    if (q->flushed != q->tail) return DDT_ERR_STATE;  // only between batches
    if (enable && !q->resp_host) {
        DeviceGuard g(q->device);
        size_t n = (size_t)q->capacity;
        cudaError_t e = cudaHostAlloc((void**)&q->resp_host, n * 4, cudaHostAllocMapped);
        if (e == cudaSuccess) e = cudaHostGetDevicePointer((void**)&q->resp_dev, q->resp_host, 0);
        if (e == cudaSuccess) e = cudaMalloc(&q->done_ctr, n * 4);
        if (e == cudaSuccess) e = cudaMemset(q->done_ctr, 0, n * 4);
        if (e != cudaSuccess) return cuda_fail("response flags", e);
        std::memset(q->resp_host, 0, n * 4);
    }
    q->resp_on = enable != 0;
    return DDT_OK;
}

int64_t ddt_pack_enqueue(ddt_queue_t q, ddt_type_t t, const void* src, int64_t count, void* dst_packed) {
    return enqueue(q, OP_PACK, t, src, count, dst_packed);
}

int64_t ddt_unpack_enqueue(ddt_queue_t q, ddt_type_t t, const void* src_packed, int64_t count, void* dst) {
    return enqueue(q, OP_UNPACK, t, src_packed, count, dst);
}

int64_t ddt_enqueue_many(ddt_queue_t q, int32_t op, int64_t n, const ddt_type_t* types, const void* const* srcs,
                         const int64_t* counts, void* const* dsts, int64_t* uids_out) {
    if (!q || n < 0 || (op != DDT_OP_PACK && op != DDT_OP_UNPACK)) return DDT_ERR_ARG;
    if (n > 0 && (!types || !srcs || !counts || !dsts)) return DDT_ERR_ARG;
    const int dop = op == DDT_OP_PACK ? OP_PACK : OP_UNPACK;
    for (int64_t i = 0; i < n; i++) {
        const int64_t uid = enqueue(q, dop, types[i], srcs[i], counts[i], dsts[i]);
        if (uids_out) uids_out[i] = uid;
        if (uid < 0) return i;
    }
    return n;
}

int64_t ddt_direct_enqueue(ddt_queue_t q, ddt_type_t src_type, const void* src, int64_t src_count,
                           ddt_type_t dst_type, void* dst, int64_t dst_count) {
    if (!q || !src_type || !dst_type || src_count < 0 || dst_count < 0) return DDT_ERR_ARG;
    if (q->sticky != DDT_OK) return q->sticky;
    if (!src_type->committed || !dst_type->committed) return DDT_ERR_STATE;
    int64_t bytes = src_count * src_type->size;
    if (bytes != dst_count * dst_type->size) return DDT_ERR_SIZE_MISMATCH;
    if (bytes > 0 && (!src || !dst)) return DDT_ERR_ARG;
    if (bytes > 0 && instances_overlap(dst_type, dst_count)) return DDT_ERR_OVERLAP;
    int64_t c = claim(q);
    if (c < 0) return c;
    ReqDesc d, a;
    std::memset(&d, 0, sizeof(d));
    std::memset(&a, 0, sizeof(a));
    if (bytes > 0) {
        DeviceLayout *dls = nullptr, *dld = nullptr;
        ddt_status_t s = type_device_layout(src_type, q->device, &dls);
        if (s == DDT_OK) s = type_device_layout(dst_type, q->device, &dld);
        if (s == DDT_OK) s = build_direct(src_type, dls, src, src_count, dst_type, dld, dst, dst_count, &d, &a);
        if (s != DDT_OK) return s;
    }
    return commit_req(q, OP_DIRECT, src_type, dst_type, bytes, d, a);
}

int32_t ddt_flush(ddt_queue_t q) {
    if (!q) return DDT_ERR_ARG;
    if (q->sticky != DDT_OK) return q->sticky;
    if (q->flushed == q->tail) return 0;
    DeviceGuard g(q->device);
    // a flushed batch is one-shot (its ring slots, types and table slot are
    // reclaimed through a completion event): graphs capture persistent plans
    // (ddt_plan_*), whose tables live as long as the plan, not flushes
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(q->stream, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone) {
        set_error("ddt_flush while the queue's stream is being captured: capture ddt_plan_launch instead");
        return DDT_ERR_STATE;
    }
    int64_t moved = gather_pending(q);
    int32_t nflushed = (int32_t)(q->tail - q->flushed);
    if (!q->scratch.descs.empty()) {
        Launchable& L = q->launch;
        q->scratch.ticket = (uint64_t)(uintptr_t)q->ticket;
        make_launchable(q->scratch, true, L, q->sm_count);
        if (L.form == 3) {
            size_t tb = device_table_bytes(q->scratch);
            ddt_queue_s::HostSlot* slot = nullptr;
            ddt_status_t s = ensure_host_slot(q, tb, &slot);
            if (s != DDT_OK) return q->sticky = s;
            write_device_table(slot->p, q->scratch, L.ub, L.ticket);
            if (q->dev_cap < tb) {
                if (q->dev_table) cudaFree(q->dev_table);  // synchronizes: old table no longer in use
                size_t cap = std::max<size_t>(tb, 64 << 10);
                cudaError_t e = cudaMalloc(&q->dev_table, cap);
                if (e != cudaSuccess) {
                    q->dev_table = nullptr;
                    q->dev_cap = 0;
                    return q->sticky = cuda_fail("cudaMalloc(table)", e);
                }
                q->dev_cap = cap;
            }
            cudaError_t e = cudaMemcpyAsync(q->dev_table, slot->p, tb, cudaMemcpyHostToDevice, q->stream);
            if (e != cudaSuccess) return q->sticky = cuda_fail("table upload", e);
            cudaEventRecord(slot->ev, q->stream);
            slot->used = true;
            L.dev = q->dev_table;
        }
        int le = launch_fused(L, q->stream, 0);
        if (le != 0) return q->sticky = cuda_fail("fused kernel launch", le);
        q->stats.launches++;
        q->stats.bytes += moved;
        for (const ReqDesc& d : q->scratch.descs) q->stats.phased += d.ph ? 1 : 0;
    }
    ddt_queue_s::Batch b{q->flushed, q->tail, get_event(q)};
    cudaEventRecord(b.ev, q->stream);
    q->inflight.push_back(b);
    q->flushed = q->tail;
    q->stats.flushes++;
    return nflushed;
}

ddt_status_t ddt_query(ddt_queue_t q, int64_t uid, int32_t* state) {
    if (!q || !state || uid < 0 || uid >= q->tail) return DDT_ERR_ARG;
    DeviceGuard g(q->device);
    reclaim(q, false);
    if (uid < q->head) {
        *state = DDT_COMPLETED;
        return q->sticky;
    }
    auto& r = q->ring[(size_t)(uid % q->capacity)];
    if (r.bytes == 0) {
        *state = DDT_COMPLETED;
        return q->sticky;
    }
    // response status written by the GPU for this very request
    if (r.desc.resp && uid < q->flushed &&
        *reinterpret_cast<volatile uint32_t*>(q->resp_host + uid % q->capacity) == (uint32_t)(uid + 1)) {
        *state = DDT_COMPLETED;
        return q->sticky;
    }
    if (uid >= q->flushed) {
        *state = DDT_PENDING;
        return q->sticky;
    }
    for (auto& b : q->inflight) {
        if (uid >= b.first && uid < b.end) {
            cudaError_t e = cudaEventQuery(b.ev);
            *state = e == cudaSuccess ? DDT_COMPLETED : DDT_BUSY;
            if (e != cudaSuccess && e != cudaErrorNotReady) return cuda_fail("query", e);
            return q->sticky;
        }
    }
    *state = DDT_COMPLETED;
    return q->sticky;
}

ddt_status_t ddt_wait(ddt_queue_t q) {
    if (!q) return DDT_ERR_ARG;
    int32_t f = ddt_flush(q);
    if (f < 0) return f;
    DeviceGuard g(q->device);
    reclaim(q, true);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess && q->sticky == DDT_OK) q->sticky = cuda_fail("wait", e);
    return q->sticky;
}

}  // extern "C"

struct ddt_plan_s {
    ddt_queue_s* q = nullptr;
    Launchable launch;
    int64_t bytes = 0;
    std::vector<ddt_type_s*> types;
};

extern "C" {

ddt_status_t ddt_plan_create(ddt_queue_t q, ddt_plan_t* out) {
    if (!q || !out) return DDT_ERR_ARG;
    if (q->sticky != DDT_OK) return q->sticky;
    DeviceGuard g(q->device);
    auto* p = new (std::nothrow) ddt_plan_s();
    if (!p) return DDT_ERR_NOMEM;
    p->q = q;
    p->bytes = gather_pending(q);
    for (int64_t u = q->flushed; u < q->tail; u++) {
        auto& r = q->ring[(size_t)(u % q->capacity)];
        if (r.bytes == 0) continue;
        for (ddt_type_s* t : {r.t, r.t2})
            if (t) {
                type_retain(t);
                p->types.push_back(t);
            }
    }
    if (!q->scratch.descs.empty()) {
        q->scratch.ticket = (uint64_t)(uintptr_t)q->ticket;
        make_launchable(q->scratch, true, p->launch, q->sm_count);
        for (const ReqDesc& d : q->scratch.descs) q->stats.phased += d.ph ? 1 : 0;
        if (p->launch.form == 3) {
            std::vector<uint8_t> host(device_table_bytes(q->scratch));
            write_device_table(host.data(), q->scratch, p->launch.ub, p->launch.ticket);
            cudaError_t e = cudaMalloc(&p->launch.dev, host.size());
            if (e == cudaSuccess) e = cudaMemcpy(p->launch.dev, host.data(), host.size(), cudaMemcpyHostToDevice);
            if (e != cudaSuccess) {
                for (auto* t : p->types) type_release(t);
                cudaFree(p->launch.dev);
                delete p;
                return cuda_fail("plan table", e);
            }
        }
    }
    // the moved requests complete in the request list without a launch
    ddt_queue_s::Batch b{q->flushed, q->tail, get_event(q)};
    cudaEventRecord(b.ev, q->stream);
    q->inflight.push_back(b);
    q->flushed = q->tail;
    *out = p;
    return DDT_OK;
}

ddt_status_t ddt_plan_launch(ddt_plan_t p) {
    if (!p) return DDT_ERR_ARG;
    ddt_queue_s* q = p->q;
    if (q->sticky != DDT_OK) return q->sticky;
    if (!p->launch.total_items) return DDT_OK;
    DeviceGuard g(q->device);
    int e = launch_fused(p->launch, q->stream, 0);
    if (e) return q->sticky = cuda_fail("plan launch", e);
    q->stats.launches++;
    q->stats.bytes += p->bytes;
    return DDT_OK;
}

ddt_status_t ddt_plan_destroy(ddt_plan_t p) {
    if (!p) return DDT_ERR_ARG;
    {
        DeviceGuard g(p->q->device);
        cudaStreamSynchronize(p->q->stream);
        if (p->launch.dev) cudaFree(p->launch.dev);
    }
    for (auto* t : p->types) type_release(t);
    delete p;
    return DDT_OK;
}

ddt_status_t ddt_queue_get_stats(ddt_queue_t q, ddt_queue_stats_t* out) {
    if (!q || !out) return DDT_ERR_ARG;
    *out = q->stats;
    return DDT_OK;
}

}  // extern "C"

// accessors used by halo.cpp
namespace ddt {
int queue_device(ddt_queue_s* q) { return q->device; }
void* queue_stream(ddt_queue_s* q) { return (void*)q->stream; }
uint64_t queue_ticket(ddt_queue_s* q) { return (uint64_t)(uintptr_t)q->ticket; }
int queue_sm_count(ddt_queue_s* q) { return q->sm_count; }
ddt_status_t queue_sticky(ddt_queue_s* q) { return q->sticky; }
void queue_set_sticky(ddt_queue_s* q, ddt_status_t s) {
    if (q->sticky == DDT_OK) q->sticky = s;
}
void queue_count_launches(ddt_queue_s* q, int64_t launches, int64_t bytes) {
    q->stats.launches += launches;
    q->stats.bytes += bytes;
}
}  // namespace ddt

// ---------------------------------------------------------------- knobs
namespace ddt {
namespace {
std::mutex g_knob_mu;
std::atomic<uint64_t> g_knob_gen{1};
}  // namespace

const char* KnobSlot::get() {
    const uint64_t G = g_knob_gen.load(std::memory_order_relaxed);
    if (gen.load(std::memory_order_acquire) != G) {
        std::lock_guard<std::mutex> lk(g_knob_mu);
        if (gen.load(std::memory_order_relaxed) != G) {
            const char* v = getenv(name);
            set = v != nullptr;
            val = v ? v : "";
            gen.store(G, std::memory_order_release);
        }
    }
    return set ? val.c_str() : nullptr;
}
}  // namespace ddt

extern "C" void ddt_reload_env(void) { ddt::g_knob_gen.fetch_add(1); }
