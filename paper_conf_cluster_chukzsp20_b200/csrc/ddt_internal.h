// ddt_internal.h -- host-side internals of libddt (types, layout cache, queue).
#pragma once
#include <atomic>
#include <cstdint>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/ddt.h"
#include "device_desc.h"

namespace ddt {

// ---------------------------------------------------------------- errors
void set_error(const std::string& msg);
// Cached getenv for DDT_* knobs (see ddt_reload_env in include/ddt.h): one
// static slot per call site, re-read only after a reload (lock-free fast
// path: one relaxed load + compare).  The pointer is valid until the next
// ddt_reload_env().
struct KnobSlot {
    const char* name;
    std::atomic<uint64_t> gen{0};
    std::string val;
    bool set = false;
    explicit KnobSlot(const char* n) : name(n) {}
    const char* get();
};
#define DDT_KNOB(NAME)                                  \
    ([]() -> const char* {                              \
        static ::ddt::KnobSlot ddt_knob_slot_{NAME};    \
        return ddt_knob_slot_.get();                    \
    }())
const char* last_error();
ddt_status_t cuda_fail(const char* what, int cuda_err);

// ---------------------------------------------------------------- types
enum TypeKind { T_BASIC, T_CONTIG, T_VECTOR, T_HVECTOR, T_INDEXED, T_HINDEXED, T_SUBARRAY, T_STRUCT, T_RESIZED };

// A closed-form strided description of the typemap's contiguous segments:
// segment (i_0..i_{D-1}) (outermost first, typemap order = row-major over the
// dims) is at  base + sum_d i_d * dims[d].stride  and has seg_len bytes.
struct Dim {
    int64_t n, stride;
};
struct Form {
    int64_t base = 0;
    int64_t seg_len = 0;
    std::vector<Dim> dims;  // outermost first
    int64_t num_segments() const;
};
// Drop unit dims, merge dims whose strides chain, fold contiguous inner dims
// into the segment.  Returns false for an empty form (some n == 0 or len 0).
bool normalize(Form& f);

struct Seg {
    int64_t off, len;
};

// Per-device copy of list-layout metadata (the device-resident layout cache).
struct DeviceLayout {
    void* offsets = nullptr;  // u32 or i64
    void* lens = nullptr;     // i64 (general)
    void* prefix = nullptr;   // i64 (general)
    void* skip = nullptr;     // u32 (general): segment holding packed byte i << kSkipShift
};

struct Layout {
    int32_t kind = DDT_LAYOUT_EMPTY;
    int64_t nseg = 0;          // segments per instance
    int64_t seg_len = 0;       // strided / uniform
    Form form;                 // strided (dims <= kMaxDims)
    bool off32 = false;        // uniform: offsets fit in int32
    std::vector<int64_t> offsets, lens, prefix;  // lists (host copy)
    int align = 16;            // power of two <= 16 dividing every offset & length
    bool overlaps = false;
};

struct ddt_type_impl;
}  // namespace ddt

struct ddt_type_s {
    int kind;
    int base = -1;
    bool predefined = false;
    int64_t elem = 0;
    int64_t count = 0, blocklen = 0, stride = 0;   // contig / vector / hvector (stride in bytes for hvector)
    std::vector<int64_t> blocklens, displs;       // indexed / hindexed
    int ndims = 0, order = 0;
    std::vector<int64_t> sizes, subsizes, starts;
    ddt_type_s* old = nullptr;
    std::vector<ddt_type_s*> types;                // struct: one oldtype per block (retained)
    std::atomic<int64_t> refs{1};

    // closed-form properties (computed at construction)
    bool nonempty = false;
    int64_t size = 0, lb = 0, ub = 0, true_lb = 0, true_ub = 0;
    int64_t align = 1;    // max alignment (= size) of the basic types in the typemap (struct epsilon, R2)
    bool sticky = false;  // explicit lb / ub markers beneath (resized, subarray): no epsilon (MPI-3.1 §4.1.6)
    bool has_form = false;
    ddt::Form form;  // normalized strided form if derivable (any number of dims)

    // committed layout
    std::mutex mu;
    bool committed = false;
    ddt::Layout layout;
    std::map<int, ddt::DeviceLayout> dev;  // device ordinal -> device cache
    // lock-free fast path of type_device_layout: the last (device, cache) pair
    std::atomic<int> fast_dev{-1};
    std::atomic<ddt::DeviceLayout*> fast_dl{nullptr};
};

namespace ddt {
void type_retain(ddt_type_s* t);
void type_release(ddt_type_s* t);
// Upload list metadata to `device` if needed (caller has set the device).
ddt_status_t type_device_layout(ddt_type_s* t, int device, DeviceLayout** out);
inline int64_t type_extent(const ddt_type_s* t) { return t->ub - t->lb; }
bool instances_overlap(ddt_type_s* t, int64_t count);  // R5 for unpack / direct destinations

// ------------------------------------------------------------ kernels
// One request -> (source, destination) descriptor pair (desc.cpp).
DivU32 make_div(uint32_t d);
ddt_status_t build_request(int op, ddt_type_s* t, const DeviceLayout* dl, const void* src, const void* dst,
                           int64_t count, ReqDesc* s, ReqDesc* d);
ddt_status_t build_direct(ddt_type_s* ts, const DeviceLayout* dls, const void* src, int64_t scount, ddt_type_s* td,
                          const DeviceLayout* dld, void* dst, int64_t dcount, ReqDesc* s, ReqDesc* d);
ddt_status_t build_typed(ddt_type_s* t, const DeviceLayout* dl, const void* p, int64_t count, ReqDesc* d);
ddt_status_t rescale_desc(ReqDesc* d, int lw);
ddt_status_t build_ll(int op, ddt_type_s* t, const DeviceLayout* dl, const void* typed, const void* window,
                      int64_t count, ReqDesc* s, ReqDesc* d);
// Largest legal log2 vector width of one typed side (type layout over pointer p).
int side_lw(ddt_type_s* t, const void* p, int64_t count);
// Base address of the device allocation containing p (CUDA driver, for IPC).
ddt_status_t alloc_base(const void* p, void** base);
// Items of a descriptor at ub vectors per thread per item.
inline uint32_t desc_items(const ReqDesc& d, int ub = kUnroll) {
    uint64_t per = (uint64_t)kThreads * (uint64_t)(d.xub ? d.xub : ub);  // exchange requests carry their own
    uint64_t n = (d.nvec + per - 1) / per;
    return n ? (uint32_t)n : 1u;  // a data-free (signal / wait) request still owns one item
}

// A batch on the host: source descriptors (items come from these), their
// destination descriptors (descs[i].aux indexes aux), and exchange side info
// (empty, or one per source descriptor).
struct HostBatch {
    std::vector<ReqDesc> descs, aux;
    std::vector<XInfo> xinfo;
    std::vector<uint32_t> gm;  // group size per request (empty: no groups), see device_desc.h
    std::vector<uint32_t> order;  // explicit item table (empty: prefix search), see device_desc.h kSpreadShift
    uint64_t ticket = 0;  // device u32[2] ticket counter offered by the caller (0: static order only)
    void clear() { descs.clear(); aux.clear(); xinfo.clear(); gm.clear(); order.clear(); ticket = 0; }
    void add(ReqDesc s, const ReqDesc& d) {
        s.aux = (uint32_t)aux.size();
        aux.push_back(d);
        descs.push_back(s);
    }
};
// A batch ready to launch: carried in the kernel parameters (form 1 / 2) or
// as a device table (form 3, `dev` owned by the caller).
struct Launchable {
    int form = 0;
    std::vector<uint8_t> blob;  // ParamBatch<CAP> bytes (form 1 / 2)
    void* dev = nullptr;        // device table (form 3)
    uint32_t total_items = 0;
    int variant = 0;            // 0 generic; 1 + lw: strided-only, one vector width; 6 general lists; 7 strided-only, phased units
    int ub = kUnroll;           // vectors per thread per item
    uint64_t ticket = 0;        // dynamic item tickets in use (device counter), 0 = static order
    int grid_mode = 0;          // 0: resident grid, static item order; 1: resident grid, tickets; 2: one CTA per item
    uint32_t claim = 0;         // exchange batches: items per ticket claim (0 = one item per CTA)
};
size_t device_table_bytes(const HostBatch& b);
uint32_t write_device_table(void* dst, const HostBatch& b, int ub, uint64_t ticket = 0, uint32_t claim = 0);
// Items per thread for a batch: the largest of {4, 2, 1} that still gives
// >= 2 items per SM, so latency-bound batches use every SM.
int choose_ub(const HostBatch& b, int sm_count);
// Reorder the requests of b so that requests with equal item counts (at item
// size ub) sit together in groups of at most max_m, and fill b.gm.  Requests only
// move within maximal runs of consecutive requests of the same exchange class
// (wait? / signal?), so the exchange kernel's item order stays deadlock-free.
void group_equal_requests(HostBatch& b, int ub, int max_m = 8);
// Re-cut eligible 8-B-wide closed-form requests into phased 16-B units
// (device_desc.h kPh*).  Only batches whose every descriptor is closed-form
// are touched (they launch the strided-only kernel variants); requests that
// signal or wait (exchange flags, LL windows) keep their chunking.  Call before
// choose_ub / group_equal_requests / make_launchable (item counts change).
void phase_batch(HostBatch& b);
// Build b.order (device_desc.h kSpreadShift) for a non-exchange batch at item
// size ub; false (b unchanged) if the batch has exchange flags or exceeds the
// encoding (4096 requests, 2^20 items per request).
bool spread_items(HostBatch& b, int ub, bool allow_pair = true);
// Kernel variants that execute paired requests (fused_kernel.cu VarT::PAIR / XPAIR).
inline bool pair_variant(int v) { return v == 9 || v == 7 || v == 4; }
inline bool xpair_variant(int v) { return v == 11 || v == 12; }
bool pair_exchange_requests(HostBatch& b);
// Pair plain (non-exchange) requests walking the same short-segment lattice (device_desc.h).
void pair_requests(HostBatch& b);
// Param form if it fits (and allowed), else form 3 with `dev` left to the caller.
// force_ub > 0 fixes the item size (exchange plans: sender and receiver chunk alike).
void make_launchable(const HostBatch& b, bool allow_param, Launchable& out, int sm_count = 148, int force_ub = 0);
int launch_fused(const Launchable& l, void* stream, int grid_cap);
int launch_exchange(const Launchable& l, const XArgs& xa, void* stream, int grid_cap);
int launch_fused_form(int form, int variant, const void* param_or_table, uint32_t total_items, void* stream, int grid_cap);
int launch_exchange_form(int form, int variant, const void* param_or_table, uint32_t total_items, const XArgs& xa,
                         void* stream, int grid_cap);
int device_sm_count(int device);

// queue accessors (queue.cpp)
int queue_device(ddt_queue_s* q);
void* queue_stream(ddt_queue_s* q);
uint64_t queue_ticket(ddt_queue_s* q);  // the queue's device ticket counter (see device_desc.h)
int queue_sm_count(ddt_queue_s* q);
ddt_status_t queue_sticky(ddt_queue_s* q);
void queue_set_sticky(ddt_queue_s* q, ddt_status_t s);
void queue_count_launches(ddt_queue_s* q, int64_t launches, int64_t bytes);
ddt_status_t nccl_fail(const char* what, int r);

}  // namespace ddt
