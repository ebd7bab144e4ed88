// device_desc.h -- the device-side request descriptor and batch tables.
//
// One descriptor = one request of the paper's request list (§IV-A.1 P:189-197:
// UID, operation, origin/target buffer, cached layout entry) flattened into the
// closed-form / list parameters the fused kernel needs.  A batch table = the
// "array of requests" handed to the single fused kernel plus the work
// table built by an exclusive prefix sum over per-request item counts (SURVEY
// §8(a) a4), which maps every CTA work item to a (request, vector range) pair.
//
// A batch reaches the kernel in one of two forms:
//   * ParamBatch<CAP>: small batches travel INSIDE the kernel's parameters
//     (__grid_constant__, <= 32 KB on sm_70+ / CUDA >= 12.1): the flush is one
//     stream operation and no dependent global load precedes the data loads;
//   * a device table (BatchHeader | prefix | descs | aux | xinfo) uploaded with
//     one cudaMemcpyAsync (flush) or once (persistent plans, halo plans).
#pragma once
#include <stdint.h>

namespace ddt {

constexpr int kMaxDims = 4;          // closed-form strided dims per layout (R7)
constexpr int kThreads = 256;        // threads per CTA of the fused kernel
constexpr int kUnroll = 4;           // max vectors per thread per item (loads in flight)
constexpr int kItemVecs = kThreads * kUnroll;  // max vectors per work item
constexpr int kUnrollNarrow = 8;     // 4-B-vector batches (variant 8): twice the loads in flight
constexpr int kSegUnroll = 4;        // variant 10: whole segments per thread per item
// A batch picks ub in {1, 2, 4} vectors per thread per item: small batches use
// smaller items so that their work spreads over all 148 SMs (latency-bound
// regime), large batches use kUnroll for memory-level parallelism.

// Every request is a (source, destination) pair of descriptors: vector v is
// loaded through the source layout and stored through the destination layout.
// PACK: typed source -> contiguous destination; UNPACK: contiguous -> typed;
// DIRECT: typed -> typed (the paper's DirectIPC op; self
// messages of a halo exchange).  K_CONTIG is the packed side (offset = v * w).
enum DescOp : uint8_t { OP_PACK = 0, OP_UNPACK = 1, OP_DIRECT = 2, OP_SIGNAL = 3 };  // SIGNAL: ready / wait items, no data
enum DescKind : uint8_t { K_STRIDED = 0, K_UNIFORM32 = 1, K_UNIFORM64 = 2, K_GENERAL = 3, K_CONTIG = 4, K_LL = 5 };
// K_LL: a window in "low-latency" format (exchange plans, small messages): 8-B
// vector v lives at byte 16*v as {u32 lo, u32 epoch, u32 hi, u32 epoch}; every
// 8-byte half carries the exchange epoch, so the receiver validates the data
// itself -- no release fence, no flag (the LL idea of NCCL's protocols).
constexpr int64_t kLLMaxBytes = 512 << 10;  // messages up to this size may use LL

// Unsigned 32-bit division by a runtime constant d via a 64-bit reciprocal:
// q = umulhi64(n, ceil(2^64 / d)) is exact for n, d < 2^32 (error < 1/d);
// d == 1 is flagged by magic == 0.
struct DivU32 {
    uint32_t d;
    uint32_t pad;
    uint64_t magic;
};

struct alignas(16) ReqDesc {
    uint64_t ptr;           // base pointer of this side (MPI buffer address or packed buffer)
    uint64_t resp;          // source desc: host-mapped u32 response-status slot, 0 = none
    uint32_t nvec;          // vectors in the request (count*size / w), < 2^32
    uint8_t op;             // DescOp
    uint8_t kind;           // DescKind
    uint8_t lw;             // log2 of the vector width w in bytes (0..4)
    uint8_t ndim;           // strided dims (innermost first), K_STRIDED only
    DivU32 vps;             // vectors per segment (uniform kinds) / per instance (general)
    int64_t base;           // byte offset of segment 0 of instance 0 (strided)
    int64_t extent;         // byte stride between instances (count)
    DivU32 nseg;            // segments per instance (uniform lists)
    DivU32 radix[kMaxDims]; // strided: dim sizes, innermost first
    int64_t stride[kMaxDims];
    uint64_t list;          // device pointer: offsets (u32 / i64) for lists
    uint64_t skip;          // general: u32 skip[i] = segment holding packed byte i << kSkipShift of an instance
    uint64_t prefix;        // general: int64 exclusive packed prefix (nseg + 1 entries)
    uint32_t list_n;        // general: number of segments per instance
    uint32_t uid_lo;        // low bits of the request UID (debug / tracing)
    uint32_t aux;           // source descriptors: index of the destination descriptor in aux[]
    uint32_t resp_val;      // value written to *resp when the request's last item is done (kRespIncrement: +1)
    uint64_t done_ctr;      // device u32 counter of finished items (reset by the finishing CTA)
    uint32_t nitems;        // items of this request in its batch (set at flush)
    uint8_t ph;             // phased 16-B units (kPh*), 0 = plain vectors; see below
    uint8_t l2_64;          // 1: short segments (< kSparseSeg B) -> loads carry the .L2::64B prefetch-size hint
    uint8_t xub;            // exchange plans: this request's vectors per thread per item (0 = the batch's ub)
    uint8_t pair;           // spread plans: 1 = request r + 1 runs in this request's items (batch.cpp pair_requests)
};

// Phased units (batch.cpp phase_batch).  A closed-form request whose common
// width is 8 B only because its segments start at 8 mod 16 (halo rows begin at
// x = 1) is re-cut per segment into [8-B head] [16-B body units] [8-B tail]
// when both sides put every segment at the same phase mod 16: vector index v
// -> segment s = v / vps, unit j = v % vps (vps = units per segment); the
// body moves as 16-B accesses.  lw is 4, nvec counts units.
constexpr uint8_t kPhOn = 1, kPhHead = 2, kPhTail = 4;
// resp_val meaning "increment the device counter *resp" (NCCL_EARLY per-message
// completion counters, waited on by stream memory operations) instead of
// "store resp_val into the host-mapped slot *resp".
constexpr uint32_t kRespIncrement = 0xffffffffu;

// Sparse sides: the L2 fetches 128 B per missed line by default; a side whose
// contiguous segments are shorter than kSparseSeg bytes loads with the PTX
// prefetch-size hint .L2::64B, which halves the DRAM over-fetch of scattered
// cells (configs[2] 12-B blocks: tools/hint_probe.cu, 137 -> 100 us).
constexpr int64_t kSparseSeg = 128;

// Exchange-only side info of a descriptor (fused P2P halo kernel).
// Per item of request r:  [wait] -> move the data -> [signal].
//   remote pack   : signal = the peer's flag for this message
//   unpack        : wait   = own flag of the message (written by the sender)
//   remote direct : wait   = own "ready" slot of the peer (the peer entered this
//                   exchange, its ghosts are free), signal = the peer's done flag
//   ready         : no data; signal = own slot in the peer's ready array
//   wait          : no data; wait = own done flag of an incoming direct message
// Flags hold the exchange epoch (monotonic, never reset).
struct alignas(16) XInfo {
    uint64_t signal;        // release `epoch` here once every item of the message moved, 0 = none
    uint64_t wait;          // acquire-wait until *wait >= epoch before moving, 0 = none
    uint32_t counter;       // multi-item messages: index of the completion counter
    uint32_t nitems;        // items of the message (signal when all are done)
    int64_t parity_stride;  // window half size: the window side moves by (epoch & 1) * stride
    uint32_t per_item;      // 1: item k signals / waits on flag k (sender and receiver chunk alike)
    uint32_t fanout;        // per-message signal: number of consecutive flags to release (>= 1)
    uint32_t gpu_scope;     // 1: the flag's reader runs on this GPU -> gpu-scope release suffices
    uint32_t pad;
};
// Exchange plans chunk every message in items of kThreads * kXchgUb vectors on
// both sides, so a receiver's unpack item k depends only on the sender's pack
// item k (per-chunk flags: unpack of a message overlaps its packing).
#ifndef DDT_XCHG_UB
#define DDT_XCHG_UB 2
#endif
constexpr int kXchgUb = DDT_XCHG_UB;
// A flagged message's chunk (item) size is a function of its byte size alone,
// so sender and receiver -- whose plans differ -- chunk it identically:
// messages that may travel in LL size (<= kLLMaxBytes) use 1 vector per thread
// per item (twice the items in flight for latency-bound halos; configs[1]
// window protocol 7.3 -> 5.7 us), larger ones kXchgUb.
inline int xchg_ub_for(int64_t bytes) { return bytes <= kLLMaxBytes ? 1 : kXchgUb; }

// General lists: a CTA work item stages the prefix / offset entries of the
// segments it touches in shared memory (found through the skip table, whose
// entry i is the segment holding packed byte i << kSkipShift of an instance)
// and every thread finds its segment by a short shared-memory search -- the
// north star's "warp-level segment lookup", at CTA level.  Windows of more
// than kGenWin segments (byte-granular types) fall back to the per-vector
// global search.
constexpr int kSkipShift = 8;
constexpr int kGenWin = 1280;

// Header of a device batch table:
//   BatchHeader | uint32 prefix[nreq + 1] (16 B padded) | uint32 gm[nreq] (16 B padded, grouped only)
//   | ReqDesc src[nreq] | ReqDesc dst[naux] | XInfo[nreq]?
// Grouped batches: m consecutive requests with equal item counts n form one
// group whose m*n items interleave chunk by chunk (item j of the group = chunk
// j / m of member j % m), so the members' same-position chunks run at the same
// time -- the +x / -x faces of a halo then touch each DRAM row together.  In
// the prefix, a group's members all hold the group's first item (the binary
// search lands on the last member) and gm[r] = m for every member.
struct alignas(16) BatchHeader {
    uint32_t nreq;
    uint32_t total_items;
    uint32_t desc_offset;   // byte offsets from the header
    uint32_t aux_offset;
    uint32_t xinfo_offset;  // 0 = no exchange info
    uint32_t naux;
    uint32_t ub;            // vectors per thread per item (1, 2 or 4)
    uint32_t flags;         // bit 0: blocked item order (else cyclic over CTAs); bit 1: grouped (gm[] present)
    uint32_t order_offset;  // 0, or byte offset of the explicit item table (kBatchSpread)
    uint32_t claim;         // exchange batches: items per claim, | kXOnce = one claim per CTA (grid = ceil(items / G))
    uint64_t ticket;        // plain: 0 = static order, else device u32[2] {next, exited}; exchange: XCtrl::tick
};
// Dynamic item tickets (multi-wave plain batches): a resident-sized grid takes
// items in increasing order from an atomic counter instead of the static
// cyclic assignment, so the items in flight stay a compact window (DRAM page
// locality) however unevenly CTAs progress; the last CTA to exit resets the
// counter for the next launch (launches sharing a counter are stream-ordered:
// one counter per queue).  Used by multi-wave batches (>= kTicketMinItemsPerSM
// items per SM) of at most kTicketMaxReqs requests (batch.cpp grid_mode_for).
constexpr uint32_t kTicketMinItemsPerSM = 8;
constexpr uint32_t kTicketMaxReqs = 64;
constexpr uint32_t kBatchBlocked = 1u, kBatchGrouped = 2u;
// Items per ticket claim of a multi-wave exchange launch (resident grid).
constexpr uint32_t kXClaim = 4;
// BatchHeader::claim flag: one claim per CTA (one-wave exchange plans, grid =
// ceil(items / G) for claim = kXOnce | G).
constexpr uint32_t kXOnce = 0x80000000u;
// Spread batches (batch.cpp spread_items): an explicit item table order[item] =
// (request << kSpreadShift) | chunk, ordered so that every request's chunks are
// spread evenly over the whole launch (chunk c of a request of n items sits at
// relative position (c + 1/2) / n): all requests progress together, so the
// DRAM-activation-bound 8-B x-face cells overlap the bandwidth-bound dense
// rows instead of following them.  Non-exchange batches only.
constexpr int kSpreadShift = 20;
// Paired requests (batch.cpp pair_requests): two requests that walk the same
// lattice of short segments a few bytes apart -- the +x and -x faces of a halo
// variable touch the two ends of the same rows -- run in the same items, the
// same thread moving vector v of both (loads of both, then stores of both), so
// each DRAM row is opened once for all four x-face accesses instead of twice.

// A small batch carried in the kernel parameters.
template <int CAP>
struct alignas(16) ParamBatch {
    BatchHeader h;                 // offsets unused
    uint32_t prefix[CAP + 4];
    uint32_t gm[CAP];
    ReqDesc descs[CAP];
    ReqDesc aux[CAP];
    XInfo xinfo[CAP];
};
constexpr int kParamSmall = 8;
constexpr int kParamLarge = 32;
static_assert(sizeof(ParamBatch<kParamLarge>) <= 32000, "kernel parameter limit");

// Control block of the fused exchange kernel (device memory, zeroed at create).
//
// Item claiming and the exchange epoch (fused_kernel.cu): CTAs claim items of
// an exchange launch from the monotonic 64-bit counter `tick` (never reset), in
// item order.  Every launch of a plan takes the same, fixed number of tickets
// (its "span"): with one item per CTA (claim == 0) each of the total_items
// CTAs claims once, span = total_items; with a resident grid looping over
// chunks of `claim` items, every CTA claims until one claim lands past the
// last chunk, span = claim * (ceil(total / claim) + grid).  So ticket t
// belongs to launch t / span -- the exchange epoch is t / span + 1, on the
// device, with no exit counter, no reset and no per-launch kernel argument:
// launches are graph-capturable, and every rank (running the same sequence of
// exchanges) derives the same epoch.
struct XCtrl {
    unsigned int trace_n;         // trace records written (tracing on)
    unsigned int pad;
    unsigned long long tick;      // item tickets claimed so far (monotonic)
    unsigned long long counters[1];  // [nsend] monotonic per-message item counters
};

// One work item of the fused exchange kernel, %globaltimer stamps (ns):
// t0 item start, t1 after its wait (== t0 if none), t2 after its data moved,
// t3 after its signal (== t2 if none).
struct TraceRec {
    unsigned int cta, item, req, op;
    unsigned long long t0, t1, t2, t3;
};

// Arguments of the fused exchange kernel: fixed for the plan's lifetime (the
// epoch derives from the claimed tickets, XCtrl), so launches are graph-capturable.
struct TraceRec;
struct XArgs {
    XCtrl* ctrl;
    int* err_flag;               // host-mapped: a wait timed out
    unsigned long long timeout_ns;
    TraceRec* trace;             // 0 = tracing off
    unsigned long long trace_cap;
};

}  // namespace ddt
