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
// ddt_flush turns [flushed, Tail) into device descriptors plus an item prefix
// sum (the work table), copies the table with one cudaMemcpyAsync and issues a
// single launch; completion of a batch is a CUDA event recorded after the
// launch (response status, reading R13/R15); ring entries are recycled once
// their batch's event has fired.
#include <algorithm>
#include <cstring>
#include <deque>
#include <vector>

#include <cuda_runtime.h>

#include "ddt_internal.h"

namespace ddt {

DivU32 make_div(uint32_t d) {
    DivU32 r;
    r.d = d;
    r.pad = 0;
    r.magic = d <= 1 ? 0ull : (~0ull) / d + 1ull;
    return r;
}

static int lowbit16(uint64_t v) {
    if (v == 0) return 16;
    uint64_t a = v & (~v + 1);
    return a > 16 ? 16 : (int)a;
}

static uint64_t uabs64(int64_t v) { return v < 0 ? (uint64_t)(-(v + 1)) + 1 : (uint64_t)v; }

ddt_status_t build_desc(ddt_type_s* t, const DeviceLayout* dl, int op, const void* noncontig, const void* packed,
                        int64_t count, ReqDesc* d) {
    const Layout& L = t->layout;
    std::memset(d, 0, sizeof(*d));
    int64_t bytes = count * t->size;
    int64_t ext = type_extent(t);
    int w = L.align;
    w = std::min(w, lowbit16((uint64_t)(uintptr_t)noncontig));
    w = std::min(w, lowbit16((uint64_t)(uintptr_t)packed));
    if (count > 1) w = std::min(w, lowbit16(uabs64(ext)));
    int lw = 0;
    while ((1 << lw) < w) lw++;
    uint64_t nvec = (uint64_t)bytes >> lw;
    if (nvec >= (1ull << 32)) {
        set_error("request too large for one descriptor (>= 2^32 vectors)");
        return DDT_ERR_UNSUPPORTED;
    }
    d->noncontig = (uint64_t)(uintptr_t)noncontig;
    d->packed = (uint64_t)(uintptr_t)packed;
    d->nvec = (uint32_t)nvec;
    d->op = (uint8_t)op;
    d->lw = (uint8_t)lw;
    d->extent = ext;
    if (L.kind == DDT_LAYOUT_STRIDED) {
        Form f = L.form;
        f.dims.insert(f.dims.begin(), Dim{count, ext});
        normalize(f);
        d->kind = K_STRIDED;
        d->base = f.base;
        d->vps = make_div((uint32_t)(f.seg_len >> lw));
        if (f.dims.empty()) {
            d->ndim = 0;
            d->extent = 0;
        } else {
            int D = (int)f.dims.size();
            if (D - 1 > kMaxDims) {
                set_error("strided layout with too many dims after count folding");
                return DDT_ERR_UNSUPPORTED;
            }
            d->ndim = (uint8_t)(D - 1);
            // innermost first; the outermost dim is the final quotient
            for (int k = 0; k < D - 1; k++) {
                const Dim& x = f.dims[(size_t)(D - 1 - k)];
                d->radix[k] = make_div((uint32_t)x.n);
                d->stride[k] = x.stride;
            }
            d->extent = f.dims[0].stride;
        }
    } else if (L.kind == DDT_LAYOUT_UNIFORM_LIST) {
        d->kind = L.off32 ? K_UNIFORM32 : K_UNIFORM64;
        d->vps = make_div((uint32_t)(L.seg_len >> lw));
        d->nseg = make_div((uint32_t)L.nseg);
        d->list = (uint64_t)(uintptr_t)dl->offsets;
    } else if (L.kind == DDT_LAYOUT_GENERAL_LIST) {
        d->kind = K_GENERAL;
        d->vps = make_div((uint32_t)(t->size >> lw));  // vectors per instance
        d->list = (uint64_t)(uintptr_t)dl->offsets;
        d->lens = (uint64_t)(uintptr_t)dl->lens;
        d->prefix = (uint64_t)(uintptr_t)dl->prefix;
        d->list_n = (uint32_t)L.nseg;
    } else {
        return DDT_ERR_STATE;
    }
    return DDT_OK;
}

}  // namespace ddt

using namespace ddt;

struct ddt_queue_s {
    struct Req {
        int64_t uid;
        int op;
        ddt_type_s* t;
        const void* src;
        void* dst;
        int64_t count;
        int64_t bytes;
        ReqDesc desc;  // built at enqueue (O(1)); flush only serializes
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
    std::vector<ReqDesc> scratch;
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

void reclaim(ddt_queue_s* q, bool block) {
    while (!q->inflight.empty()) {
        auto& b = q->inflight.front();
        cudaError_t e = block ? cudaEventSynchronize(b.ev) : cudaEventQuery(b.ev);
        if (e == cudaErrorNotReady) return;
        if (e != cudaSuccess && q->sticky == DDT_OK) q->sticky = cuda_fail("batch completion", e);
        for (int64_t u = b.first; u < b.end; u++) {
            auto& r = q->ring[(size_t)(u % q->capacity)];
            type_release(r.t);
            r.t = nullptr;
        }
        q->head = b.end;
        q->event_pool.push_back(b.ev);
        q->inflight.pop_front();
    }
}

int64_t enqueue(ddt_queue_s* q, int op, ddt_type_s* t, const void* src, int64_t count, void* dst) {
    if (!q || !t || count < 0) return DDT_ERR_ARG;
    if (q->sticky != DDT_OK) return q->sticky;
    if (!t->committed) return DDT_ERR_STATE;
    int64_t bytes = count * t->size;
    if (bytes > 0 && (!src || !dst)) return DDT_ERR_ARG;
    if (op == OP_UNPACK && bytes > 0 && t->layout.overlaps) return DDT_ERR_OVERLAP;
    if (q->tail - q->head >= q->capacity) {
        DeviceGuard g(q->device);
        reclaim(q, false);
        if (q->tail - q->head >= q->capacity) return DDT_ERR_QUEUE_FULL;  // negative UID
    }
    ReqDesc desc;
    if (bytes > 0) {
        DeviceGuard g(q->device);
        DeviceLayout* dl = nullptr;
        ddt_status_t s = type_device_layout(t, q->device, &dl);
        if (s != DDT_OK) return s;
        const void* nc = op == OP_PACK ? src : dst;
        const void* pk = op == OP_PACK ? dst : src;
        s = build_desc(t, dl, op, nc, pk, count, &desc);
        if (s != DDT_OK) return s;
    }
    int64_t uid = q->tail++;
    auto& r = q->ring[(size_t)(uid % q->capacity)];
    r.desc = desc;
    r.desc.uid_lo = (uint32_t)uid;
    r.uid = uid;
    r.op = op;
    r.t = t;
    type_retain(t);
    r.src = src;
    r.dst = dst;
    r.count = count;
    r.bytes = bytes;
    q->stats.requests++;
    return uid;
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

}  // namespace

namespace ddt {
// Serialize a batch table: header | item prefix | descriptors.
size_t table_bytes(size_t nreq) {
    size_t pre = ((nreq + 1) * 4 + 15) & ~(size_t)15;
    return sizeof(BatchHeader) + pre + nreq * sizeof(ReqDesc);
}
uint32_t write_table(void* dst, const ReqDesc* descs, size_t nreq) {
    auto* h = (BatchHeader*)dst;
    size_t pre = ((nreq + 1) * 4 + 15) & ~(size_t)15;
    auto* prefix = (uint32_t*)((char*)dst + sizeof(BatchHeader));
    uint64_t acc = 0;
    for (size_t i = 0; i < nreq; i++) {
        prefix[i] = (uint32_t)acc;
        acc += desc_items(descs[i]);
    }
    prefix[nreq] = (uint32_t)acc;
    h->nreq = (uint32_t)nreq;
    h->total_items = (uint32_t)acc;
    h->desc_offset = (uint32_t)(sizeof(BatchHeader) + pre);
    h->pad = 0;
    std::memcpy((char*)dst + h->desc_offset, descs, nreq * sizeof(ReqDesc));
    return (uint32_t)acc;
}
}  // namespace ddt

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
    }
    *out = q;
    return DDT_OK;
}

ddt_status_t ddt_queue_destroy(ddt_queue_t q) {
    if (!q) return DDT_ERR_ARG;
    {
        DeviceGuard g(q->device);
        reclaim(q, true);
        for (int64_t u = q->flushed; u < q->tail; u++) type_release(q->ring[(size_t)(u % q->capacity)].t);
        for (auto e : q->event_pool) cudaEventDestroy(e);
        for (auto& s : q->slots) {
            if (s.p) cudaFreeHost(s.p);
            if (s.ev) cudaEventDestroy(s.ev);
        }
        if (q->dev_table) cudaFree(q->dev_table);
    }
    delete q;
    return DDT_OK;
}

int64_t ddt_pack_enqueue(ddt_queue_t q, ddt_type_t t, const void* src, int64_t count, void* dst_packed) {
    return enqueue(q, OP_PACK, t, src, count, dst_packed);
}

int64_t ddt_unpack_enqueue(ddt_queue_t q, ddt_type_t t, const void* src_packed, int64_t count, void* dst) {
    return enqueue(q, OP_UNPACK, t, src_packed, count, dst);
}

int32_t ddt_flush(ddt_queue_t q) {
    if (!q) return DDT_ERR_ARG;
    if (q->sticky != DDT_OK) return q->sticky;
    if (q->flushed == q->tail) return 0;
    DeviceGuard g(q->device);
    auto& descs = q->scratch;
    descs.clear();
    int64_t moved = 0;
    for (int64_t u = q->flushed; u < q->tail; u++) {
        auto& r = q->ring[(size_t)(u % q->capacity)];
        if (r.bytes == 0) continue;
        descs.push_back(r.desc);
        moved += r.bytes;
    }
    int32_t nflushed = (int32_t)(q->tail - q->flushed);
    if (!descs.empty()) {
        size_t tb = table_bytes(descs.size());
        ddt_queue_s::HostSlot* slot = nullptr;
        ddt_status_t s = ensure_host_slot(q, tb, &slot);
        if (s != DDT_OK) return q->sticky = s;
        uint32_t items = write_table(slot->p, descs.data(), descs.size());
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
        int le = launch_fused(q->dev_table, items, q->stream, 0);
        if (le != 0) return q->sticky = cuda_fail("fused kernel launch", le);
        q->stats.launches++;
        q->stats.bytes += moved;
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
    void* table = nullptr;
    uint32_t items = 0;
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
    std::vector<ReqDesc> descs;
    for (int64_t u = q->flushed; u < q->tail; u++) {
        auto& r = q->ring[(size_t)(u % q->capacity)];
        if (r.bytes == 0) continue;
        descs.push_back(r.desc);
        p->bytes += r.bytes;
        type_retain(r.t);
        p->types.push_back(r.t);
    }
    if (!descs.empty()) {
        std::vector<uint8_t> host(table_bytes(descs.size()));
        p->items = write_table(host.data(), descs.data(), descs.size());
        cudaError_t e = cudaMalloc(&p->table, host.size());
        if (e == cudaSuccess) e = cudaMemcpy(p->table, host.data(), host.size(), cudaMemcpyHostToDevice);
        if (e != cudaSuccess) {
            for (auto* t : p->types) type_release(t);
            cudaFree(p->table);
            delete p;
            return cuda_fail("plan table", e);
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
    if (!p->items) return DDT_OK;
    DeviceGuard g(q->device);
    int e = launch_fused(p->table, p->items, q->stream, 0);
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
        cudaFree(p->table);
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
