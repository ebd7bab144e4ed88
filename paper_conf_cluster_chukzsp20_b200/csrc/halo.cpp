// halo.cpp -- persistent halo-exchange plans (ddt_halo_create / ddt_exchange).
//
// Paper: Alg 3 -- one MPI_Isend / MPI_Irecv per boundary buffer,
// the runtime packs and unpacks implicitly; §IV-B -- the sender
// enqueues packing and sends once a pack completes, the receiver
// enqueues unpacking on arrival, and pack, unpack and DirectIPC may be
// fused into one kernel.  Domain decomposition (Fig. 3) is the
// only parallelism in the paper.
//
// B200 realisation:
//   NCCL mode: fused pack launch (all outgoing messages, per-peer contiguous
//     staging ordered by tag; self messages straight into the receive staging)
//     -> ncclGroupStart / {ncclSend, ncclRecv} per remote peer / ncclGroupEnd
//     over NVLink 5 -> fused unpack launch.  Work tables are built once here.
//   P2P mode: ONE kernel: pack stores go straight into the peer's window
//     (CUDA IPC mapping, NVSwitch), a per-message epoch flag is released when
//     the message is complete, unpack work waits on its flag (see
//     fused_kernel.cu).  Windows are double-buffered by iteration parity;
//     this requires a symmetric pattern (every peer we send to sends to us),
//     which is checked here.
//   Both: a one-time metadata exchange over NCCL validates that every send
//   matches the peer's receive of the same tag and size (DDT_ERR_SIZE_MISMATCH)
//   and tells each sender where its messages land; iterations can be replayed
//   from a CUDA graph captured on first use.
#include <algorithm>
#include <cstddef>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <tuple>
#include <vector>

#include <cuda.h>
#include <cuda_runtime.h>

#include "ddt_internal.h"
#include "nccl_min.h"

using namespace ddt;

namespace {

constexpr int64_t kAlign = 16;

int64_t round_up(int64_t v, int64_t a) { return (v + a - 1) / a * a; }

// Receive-side layout shared by the window (P2P) and the receive staging (NCCL).
struct RecvLayout {
    std::vector<int> order;          // recv indices sorted by (peer, tag)
    std::vector<int64_t> data_off;   // per recv index: offset inside one parity half
    std::vector<int> flag_idx;       // per recv index: first of its per-chunk flag slots
    std::vector<int> lw;             // per recv index: vector width of the unpack side
    std::vector<int> nflags;         // per recv index: chunks (items at kXchgUb) of the message
    std::vector<int> ll_ok;          // per recv index: window space reserved for the LL format
    int64_t ready_off = 0;           // byte offset of the per-sender "ready" slots (pack-free mode)
    int64_t flags_bytes = 0, parity_stride = 0, window_bytes = 0;
};

// Item size (vectors per thread) of a flagged / LL exchange message: a
// function of its byte size (and of one run-wide knob), so the sender and the
// receiver -- whose plans differ -- chunk it identically (device_desc.h
// xchg_ub_for).  DDT_XUB_SMALL: experiments (messages <= kLLMaxBytes).
int xub_for(int64_t bytes) {
    const char* e = DDT_KNOB("DDT_XUB_SMALL");
    if (bytes <= kLLMaxBytes && e && (e[0] == '1' || e[0] == '2')) return e[0] - '0';
    return xchg_ub_for(bytes);
}

// reserve_ll: window space for the LL format (P2P window mode only; the NCCL
// staging must not carry the gaps -- they would be transferred).
RecvLayout layout_recvs(int32_t nrecv, const ddt_recv_t* recvs, bool reserve_ll = true) {
    RecvLayout L;
    L.order.resize((size_t)nrecv);
    for (int i = 0; i < nrecv; i++) L.order[(size_t)i] = i;
    std::sort(L.order.begin(), L.order.end(), [&](int a, int b) {
        return std::make_pair(recvs[a].peer, recvs[a].tag) < std::make_pair(recvs[b].peer, recvs[b].tag);
    });
    L.data_off.assign((size_t)nrecv, 0);
    L.flag_idx.assign((size_t)nrecv, 0);
    L.lw.assign((size_t)nrecv, 0);
    L.nflags.assign((size_t)nrecv, 1);
    L.ll_ok.assign((size_t)nrecv, 0);
    int64_t off = 0, nflag = 0;
    for (size_t k = 0; k < L.order.size(); k++) {
        int i = L.order[k];
        int64_t bytes = recvs[i].count * recvs[i].type->size;
        const int64_t chunk = (int64_t)kThreads * xub_for(bytes);  // vectors per exchange item
        off = round_up(off, kAlign);
        L.data_off[(size_t)i] = off;
        int lw = recvs[i].type->committed ? std::min(4, side_lw(recvs[i].type, recvs[i].buf, recvs[i].count)) : 0;
        L.lw[(size_t)i] = lw;
        L.nflags[(size_t)i] = (int)std::max<int64_t>(1, ((bytes >> lw) + chunk - 1) / chunk);
        L.flag_idx[(size_t)i] = (int)nflag;
        nflag += L.nflags[(size_t)i];
        // small messages of 8-B-capable layouts may travel in LL format (2x the bytes)
        L.ll_ok[(size_t)i] = (reserve_ll && lw >= 3 && bytes <= kLLMaxBytes && bytes % 8 == 0) ? 1 : 0;
        off += L.ll_ok[(size_t)i] ? 2 * bytes : bytes;
    }
    int64_t nready = 0;  // one slot per possible sender rank
    for (int i = 0; i < nrecv; i++) nready = std::max<int64_t>(nready, (int64_t)recvs[i].peer + 1);
    L.ready_off = 8 * nflag;
    L.flags_bytes = round_up(std::max<int64_t>(8 * (nflag + nready), 8), 256);
    L.parity_stride = round_up(std::max<int64_t>(off, 16), 256);
    L.window_bytes = L.flags_bytes + 2 * L.parity_stride;
    return L;
}

struct DirEntry {
    int64_t tag, bytes, data_off, flag_idx, lw, nflags, ll_ok;
    // pack-free mode: where the receive buffer lives and how it is laid out
    int64_t ipc[8];      // cudaIpcMemHandle_t of the buffer's allocation
    int64_t alloc_off;   // buffer address - allocation base
    ReqDesc desc;        // receiver's typed descriptor (ptr = 0), at its widest legal width
};
struct Directory {  // what a receiver tells one sender
    int64_t parity_stride = 0, data_base = 0, ready_base = 0, direct = 0;
    std::vector<DirEntry> e;  // sorted by tag
};
constexpr int kDescWords = (int)(sizeof(ReqDesc) / 8);
static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");

struct Xfer {
    int peer;
    int64_t send_off, send_bytes;  // in send staging
    int64_t recv_off, recv_bytes;  // in receive staging
};

}  // namespace

struct ddt_halo_s {
    ddt_queue_s* q = nullptr;
    int device = 0;
    cudaStream_t stream = nullptr;
    int rank = 0, nranks = 1, mode = DDT_XCHG_NCCL;
    void* comm = nullptr;
    ddt_allgather_fn ag = nullptr;  // host all-gather for plan metadata (else NCCL)
    void* ag_ctx = nullptr;
    std::vector<ddt_send_t> sends;
    std::vector<ddt_recv_t> recvs;
    // NCCL mode
    void* send_stage = nullptr;
    void* recv_stage = nullptr;
    std::vector<Xfer> xfers;
    bool self_nccl = false;       // test hook DDT_SELF_VIA_NCCL: self messages through staging + NCCL
    // NCCL_EARLY: per remote peer, its stream, its messages' completion counters
    // (indices into early_ctr) and the event joining it back into the queue stream
    struct EarlyPeer {
        size_t xfer;
        std::vector<int> ctr;
        cudaStream_t s = nullptr;
        cudaEvent_t done = nullptr;
    };
    bool early = false;
    std::vector<EarlyPeer> epeers;
    uint32_t* early_ctr = nullptr;   // device: per remote pack request, completions since the last reset
    uint32_t* early_done = nullptr;  // device: per remote pack request, finished items (kernel bookkeeping)
    cudaEvent_t early_start = nullptr;
    Launchable pack_l, unpack_l;  // NCCL mode: pack (+ direct self copies), unpack
    // P2P mode
    Launchable x_l;               // P2P mode: the single fused exchange kernel
    void* ctrl = nullptr;
    int* err_host = nullptr;
    int* err_dev = nullptr;
    uint64_t timeout_ns = 10ull * 1000 * 1000 * 1000;
    int grid_cap = 0;
    bool x_flags = false;         // P2P plan has remote messages (flags); else the plain fused kernel runs
    void* trace = nullptr;        // device TraceRec buffer (tracing on) and its capacity
    int64_t trace_cap = 0;
    std::vector<void*> ipc_opened;  // peers' receive buffers mapped for pack-free writes
    // graph replay
    bool use_graph = false;
    cudaGraphExec_t gexec = nullptr;
    int32_t launches = 0;
    int64_t bytes = 0;
};

namespace {

struct DevGuard {
    int prev = -1;
    explicit DevGuard(int d) {
        cudaGetDevice(&prev);
        if (prev != d) cudaSetDevice(d);
    }
    ~DevGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

ddt_status_t upload(const std::vector<uint8_t>& host, void** dev) {
    cudaError_t e = cudaMalloc(dev, std::max<size_t>(host.size(), 16));
    if (e != cudaSuccess) return cuda_fail("cudaMalloc(halo)", e);
    e = cudaMemcpy(*dev, host.data(), host.size(), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return cuda_fail("cudaMemcpy(halo)", e);
    return DDT_OK;
}

// Small batches ride in the kernel parameters (captured into the graph node);
// larger ones are uploaded once as a device table.  Requests of equal size are
// grouped (interleaved chunk by chunk) first, at the item size the table uses,
// when the batch spans several waves of CTAs: only then would the members
// otherwise run at different times (measured: COMB 139 -> 124 us; a one-wave
// batch such as configs[1] only pays the extra lookup, 3.5 -> 3.75 us).
ddt_status_t make_table(HostBatch& b, Launchable& l, int sm_count, int force_ub = 0) {
    phase_batch(b);
    int ub = force_ub > 0 ? force_ub : choose_ub(b, sm_count);
    uint64_t items = 0;
    for (const auto& d : b.descs) items += desc_items(d, ub);
    const char* ga = DDT_KNOB("DDT_GROUP_ALWAYS");  // tests: exercise grouping on small plans
    const char* sp = DDT_KNOB("DDT_SPREAD");  // 0: group equal requests instead of spreading every request
    const char* sa = DDT_KNOB("DDT_SPREAD_ALWAYS");  // tests: spread (and pair) small plans too
    const bool many = items > 8ull * (uint64_t)sm_count || (sa && sa[0] == '1' && force_ub <= 0);
    bool spread = false;
    if (many && !(sp && sp[0] == '0')) {
        // spread plans run one CTA per item (batch.cpp grid_mode_for): with one
        // vector per thread they get the most CTAs in flight and the one-slot
        // kernel (variant 9 for phased batches) -- COMB P = 1 116.6 -> 101.6 us
        // -- when some request has short segments (x faces: DRAM-access bound);
        // all-dense plans keep the large items (COMB dense faces alone: 16 us at
        // ub 4, 28.5 us at ub 1)
        bool sparse = false;
        for (const ReqDesc& d : b.descs) sparse |= d.l2_64 || b.aux[d.aux].l2_64;
        const char* su = DDT_KNOB("DDT_SPREAD_UB");  // experiments: item size of spread plans
        const int sub = force_ub > 0 ? ub : (su ? std::max(1, std::min(4, atoi(su))) : (sparse ? 1 : ub));
        // dense requests of a sparse plan may keep larger items of their own
        // (ReqDesc::xub): DDT_SPREAD_DENSE_UB (experiments)
        const char* du = DDT_KNOB("DDT_SPREAD_DENSE_UB");
        const int dub = du ? std::max(0, std::min(4, atoi(du))) : 0;
        if (sparse && dub > sub && force_ub <= 0)
            for (ReqDesc& d : b.descs)
                if (!d.l2_64 && !b.aux[d.aux].l2_64 && d.op != OP_SIGNAL) d.xub = (uint8_t)dub;
        spread = spread_items(b, sub);
        // undo the dense item sizes set above (only those: an exchange plan's
        // xub is part of its protocol -- the receiver's chunk flags and the
        // message counters assume xub_for's chunking)
        if (!spread && force_ub <= 0)
            for (ReqDesc& d : b.descs) d.xub = 0;
        if (spread) ub = sub;
    }
    // multi-wave exchange plans: pair +x / -x style packs and unpacks
    // (fused_kernel.cu run_pair_x; COMB window proxy 178 -> 144 us); one-wave
    // (latency-bound) plans keep one request per item (configs[1] window
    // proxy: 4.35 us unpaired, 6.35 us paired)
    const char* xpa = DDT_KNOB("DDT_XPAIR_ALWAYS");  // tests: pair one-wave exchange plans too
    const bool xpaired = force_ub > 0 && (many || (xpa && xpa[0] == '1')) && pair_exchange_requests(b);
    // one-wave plain plans pair their +x / -x requests only on request
    // (DDT_PAIR1=1: configs[1] 1.99 -> 2.32 us when paired)
    const char* p1 = DDT_KNOB("DDT_PAIR1");
    if (!spread && force_ub <= 0 && !many && p1 && p1[0] == '1') pair_requests(b);
    bool ppaired = false;
    for (const ReqDesc& d : b.descs) ppaired |= !spread && !xpaired && d.pair != 0;
    if (!spread && !xpaired && !ppaired && (many || (ga && ga[0] == '1'))) group_equal_requests(b, ub);
    for (ReqDesc& d : b.descs)  // response slots: the finishing CTA compares its count with the item count
        if (d.resp) d.nitems = desc_items(d, ub);
    make_launchable(b, !spread, l, sm_count, ub);
    bool paired = false;
    for (const ReqDesc& d : b.descs) paired |= d.pair != 0;
    if (paired && xpaired && !xpair_variant(l.variant)) {  // the exchange instance cannot run pairs: undo them
        for (ReqDesc& d : b.descs) d.pair = 0;
        if (many || (ga && ga[0] == '1')) group_equal_requests(b, ub);
        make_launchable(b, true, l, sm_count, ub);
    } else if (paired && !xpaired && (l.form == 3 ? !pair_variant(l.variant) : l.variant != 9)) {
        // the chosen instance cannot run pairs (parameter batches: the one-slot instance only): undo them
        for (ReqDesc& d : b.descs) d.pair = 0;
        if (spread) spread_items(b, ub, false);
        make_launchable(b, !spread, l, sm_count, ub);
    }
    if (l.form != 3) return DDT_OK;
    std::vector<uint8_t> host(device_table_bytes(b));
    write_device_table(host.data(), b, l.ub, l.ticket, l.claim);
    return upload(host, &l.dev);
}

// Exchange every receiver->sender directory over NCCL (nranks > 1), then agree
// on a status with an all-reduce(min) so that all ranks fail or succeed together.
ddt_status_t exchange_directories(ddt_halo_s* h, const std::vector<std::vector<int64_t>>& out,
                                  std::vector<std::vector<int64_t>>& in) {
    const NcclApi* n = nccl();
    if (!n) {
        set_error("NCCL not available for the halo metadata exchange");
        return DDT_ERR_UNSUPPORTED;
    }
    int P = h->nranks;
    in.assign((size_t)P, {});
    std::vector<int64_t> cnt_out((size_t)P, 0), cnt_in((size_t)P, 0);
    for (int p = 0; p < P; p++) cnt_out[(size_t)p] = (int64_t)out[(size_t)p].size();
    int64_t* d_cnt = nullptr;
    cudaError_t e = cudaMalloc(&d_cnt, 2 * sizeof(int64_t) * (size_t)P);
    if (e != cudaSuccess) return cuda_fail("cudaMalloc(meta)", e);
    cudaMemcpy(d_cnt, cnt_out.data(), sizeof(int64_t) * (size_t)P, cudaMemcpyHostToDevice);
    int r = n->GroupStart();
    for (int p = 0; p < P && r == 0; p++) {
        if (p == h->rank) continue;
        r = n->Send(d_cnt + p, 8, kNcclUint8, p, h->comm, h->stream);
        if (r == 0) r = n->Recv(d_cnt + P + p, 8, kNcclUint8, p, h->comm, h->stream);
    }
    int r2 = n->GroupEnd();
    if (r == 0) r = r2;
    if (r != 0) {
        cudaFree(d_cnt);
        return nccl_fail("halo metadata (counts)", r);
    }
    cudaStreamSynchronize(h->stream);
    cudaMemcpy(cnt_in.data(), d_cnt + P, sizeof(int64_t) * (size_t)P, cudaMemcpyDeviceToHost);
    cudaFree(d_cnt);
    int64_t tot_out = 0, tot_in = 0;
    for (int p = 0; p < P; p++) {
        if (p == h->rank) continue;
        tot_out += cnt_out[(size_t)p];
        tot_in += cnt_in[(size_t)p];
    }
    int64_t* d_buf = nullptr;
    e = cudaMalloc(&d_buf, sizeof(int64_t) * (size_t)std::max<int64_t>(tot_out + tot_in, 1));
    if (e != cudaSuccess) return cuda_fail("cudaMalloc(meta)", e);
    std::vector<int64_t> flat_out;
    for (int p = 0; p < P; p++)
        if (p != h->rank) flat_out.insert(flat_out.end(), out[(size_t)p].begin(), out[(size_t)p].end());
    if (tot_out) cudaMemcpy(d_buf, flat_out.data(), sizeof(int64_t) * (size_t)tot_out, cudaMemcpyHostToDevice);
    r = n->GroupStart();
    int64_t oo = 0, io = tot_out;
    for (int p = 0; p < P && r == 0; p++) {
        if (p == h->rank) continue;
        if (cnt_out[(size_t)p]) r = n->Send(d_buf + oo, (size_t)cnt_out[(size_t)p] * 8, kNcclUint8, p, h->comm, h->stream);
        if (r == 0 && cnt_in[(size_t)p])
            r = n->Recv(d_buf + io, (size_t)cnt_in[(size_t)p] * 8, kNcclUint8, p, h->comm, h->stream);
        oo += cnt_out[(size_t)p];
        io += cnt_in[(size_t)p];
    }
    r2 = n->GroupEnd();
    if (r == 0) r = r2;
    if (r != 0) {
        cudaFree(d_buf);
        return nccl_fail("halo metadata (directories)", r);
    }
    cudaStreamSynchronize(h->stream);
    std::vector<int64_t> flat_in((size_t)tot_in);
    if (tot_in)
        cudaMemcpy(flat_in.data(), d_buf + tot_out, sizeof(int64_t) * (size_t)tot_in, cudaMemcpyDeviceToHost);
    cudaFree(d_buf);
    io = 0;
    for (int p = 0; p < P; p++) {
        if (p == h->rank) continue;
        in[(size_t)p].assign(flat_in.begin() + io, flat_in.begin() + io + cnt_in[(size_t)p]);
        io += cnt_in[(size_t)p];
    }
    return DDT_OK;
}

// Host path: every rank all-gathers one blob = concat over destination p of
// (len_p, directory_p...); rank r keeps section r of every peer's blob.
ddt_status_t exchange_directories_host(ddt_halo_s* h, const std::vector<std::vector<int64_t>>& out,
                                       std::vector<std::vector<int64_t>>& in) {
    const int P = h->nranks;
    std::vector<int64_t> blob;
    for (int p = 0; p < P; p++) {
        blob.push_back((int64_t)out[(size_t)p].size());
        blob.insert(blob.end(), out[(size_t)p].begin(), out[(size_t)p].end());
    }
    int64_t mine = (int64_t)blob.size();
    std::vector<int64_t> sizes((size_t)P);
    if (h->ag(h->ag_ctx, &mine, 8, sizes.data()) != 0) {
        set_error("host all-gather failed (sizes)");
        return DDT_ERR_ARG;
    }
    int64_t mx = *std::max_element(sizes.begin(), sizes.end());
    blob.resize((size_t)mx, 0);
    std::vector<int64_t> all((size_t)(mx * P));
    if (h->ag(h->ag_ctx, blob.data(), mx * 8, all.data()) != 0) {
        set_error("host all-gather failed (directories)");
        return DDT_ERR_ARG;
    }
    in.assign((size_t)P, {});
    for (int q = 0; q < P; q++) {
        const int64_t* b = all.data() + (size_t)q * (size_t)mx;
        int64_t pos = 0;
        for (int p = 0; p < P; p++) {
            int64_t len = b[pos++];
            if (p == h->rank) in[(size_t)q].assign(b + pos, b + pos + len);
            pos += len;
        }
    }
    return DDT_OK;
}

ddt_status_t agree(ddt_halo_s* h, ddt_status_t mine) {
    if (h->nranks == 1) return mine;
    if (h->ag) {
        std::vector<int32_t> all((size_t)h->nranks);
        int32_t v = mine;
        if (h->ag(h->ag_ctx, &v, 4, all.data()) != 0) return DDT_ERR_ARG;
        return *std::min_element(all.begin(), all.end());
    }
    const NcclApi* n = nccl();
    if (!n) return DDT_ERR_UNSUPPORTED;
    int32_t* d = nullptr;
    if (cudaMalloc(&d, 8) != cudaSuccess) return DDT_ERR_CUDA;
    int32_t v = mine;
    cudaMemcpy(d, &v, 4, cudaMemcpyHostToDevice);
    int r = n->AllReduce(d, d + 1, 1, kNcclInt32, kNcclMin, h->comm, h->stream);
    cudaStreamSynchronize(h->stream);
    int32_t res = DDT_OK;
    cudaMemcpy(&res, d + 1, 4, cudaMemcpyDeviceToHost);
    cudaFree(d);
    if (r != 0) return nccl_fail("halo status all-reduce", r);
    return res;
}

// [n, parity_stride, data_base, ready_base, direct] then n entries of
// [tag, bytes, data_off, flag_idx, lw, nflags, ll_ok] (+ [ipc x8, alloc_off, desc x kDescWords] if direct)
Directory parse_dir(const std::vector<int64_t>& v) {
    Directory d;
    if (v.size() < 5) return d;
    int64_t n = v[0];
    d.parity_stride = v[1];
    d.data_base = v[2];
    d.ready_base = v[3];
    d.direct = v[4];
    size_t pos = 5;
    const size_t stride = 7 + (d.direct ? 9 + kDescWords : 0);
    for (int64_t i = 0; i < n && pos + stride <= v.size(); i++, pos += stride) {
        DirEntry e{};
        e.tag = v[pos];
        e.bytes = v[pos + 1];
        e.data_off = v[pos + 2];
        e.flag_idx = v[pos + 3];
        e.lw = v[pos + 4];
        e.nflags = v[pos + 5];
        e.ll_ok = v[pos + 6];
        if (d.direct) {
            std::memcpy(e.ipc, &v[pos + 7], 64);
            e.alloc_off = v[pos + 15];
            std::memcpy(&e.desc, &v[pos + 16], sizeof(ReqDesc));
        }
        d.e.push_back(e);
    }
    return d;
}

void free_halo(ddt_halo_s* h) {
    if (h->gexec) cudaGraphExecDestroy(h->gexec);
    for (auto& p : h->epeers) {
        if (p.s) cudaStreamDestroy(p.s);
        if (p.done) cudaEventDestroy(p.done);
    }
    if (h->early_start) cudaEventDestroy(h->early_start);
    cudaFree(h->early_ctr);
    cudaFree(h->early_done);
    cudaFree(h->send_stage);
    cudaFree(h->recv_stage);
    cudaFree(h->pack_l.dev);
    cudaFree(h->unpack_l.dev);
    cudaFree(h->x_l.dev);
    cudaFree(h->ctrl);
    if (h->err_host) cudaFreeHost(h->err_host);
    for (void* p : h->ipc_opened) cudaIpcCloseMemHandle(p);
    for (auto& s : h->sends) type_release(s.type);
    for (auto& r : h->recvs) type_release(r.type);
    delete h;
}

// Stream memory operations (driver API, bound through the runtime's entry
// point query: no link-time libcuda dependency).
typedef CUresult (*WaitValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*WriteValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
struct MemOps {
    WaitValue32Fn wait = nullptr;
    WriteValue32Fn write = nullptr;
};
const MemOps* memops() {
    static MemOps m;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q1, q2;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue32", (void**)&m.wait, cudaEnableDefault, &q1) != cudaSuccess ||
            q1 != cudaDriverEntryPointSuccess)
            m.wait = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", (void**)&m.write, cudaEnableDefault, &q2) != cudaSuccess ||
            q2 != cudaDriverEntryPointSuccess)
            m.write = nullptr;
    });
    return (m.wait && m.write) ? &m : nullptr;
}

// NCCL_EARLY transfer: every remote peer's send/recv group on its own stream,
// started once that peer's pack requests have completed.  Groups
// are issued in increasing peer order on every rank (a consistent order of
// rank pairs: no deadlock even when NCCL serialises a communicator's kernels).
ddt_status_t record_early_transfer(ddt_halo_s* h) {
    const NcclApi* n = nccl();
    const MemOps* mo = memops();
    if (!n || !mo) return DDT_ERR_UNSUPPORTED;
    for (auto& P : h->epeers) {
        cudaError_t e = cudaStreamWaitEvent(P.s, h->early_start, 0);  // after the work preceding this exchange
        if (e != cudaSuccess) return cuda_fail("early send: stream wait", e);
        for (int k : P.ctr) {  // this peer's messages are packed (counter set by the finishing CTA)
            CUresult r = mo->wait((CUstream)P.s, (CUdeviceptr)(uintptr_t)(h->early_ctr + k), 1u,
                                  CU_STREAM_WAIT_VALUE_GEQ);
            if (r != CUDA_SUCCESS) return cuda_fail("early send: cuStreamWaitValue32", cudaErrorUnknown);
        }
        for (int k : P.ctr) {  // re-arm for the next exchange (ordered before its pack by the join below)
            CUresult r = mo->write((CUstream)P.s, (CUdeviceptr)(uintptr_t)(h->early_ctr + k), 0u, 0);
            if (r != CUDA_SUCCESS) return cuda_fail("early send: cuStreamWriteValue32", cudaErrorUnknown);
        }
        const Xfer& x = h->xfers[P.xfer];
        int r = n->GroupStart();
        if (r == 0 && x.send_bytes)
            r = n->Send((char*)h->send_stage + x.send_off, (size_t)x.send_bytes, kNcclUint8, x.peer, h->comm, P.s);
        if (r == 0 && x.recv_bytes)
            r = n->Recv((char*)h->recv_stage + x.recv_off, (size_t)x.recv_bytes, kNcclUint8, x.peer, h->comm, P.s);
        int r2 = n->GroupEnd();
        if (r == 0) r = r2;
        if (r != 0) return nccl_fail("halo send/recv (early)", r);
        e = cudaEventRecord(P.done, P.s);
        if (e != cudaSuccess) return cuda_fail("early send: event", e);
    }
    for (auto& P : h->epeers) {
        cudaError_t e = cudaStreamWaitEvent(h->stream, P.done, 0);
        if (e != cudaSuccess) return cuda_fail("early send: join", e);
    }
    return DDT_OK;
}

ddt_status_t record_exchange(ddt_halo_s* h) {
    if (h->mode != DDT_XCHG_NCCL) {
        int e;
        if (h->x_flags) {
            XArgs xa{};  // the epoch is device-resident (XCtrl::epoch): nothing here varies per launch
            xa.ctrl = reinterpret_cast<XCtrl*>(h->ctrl);
            xa.err_flag = h->err_dev;
            xa.timeout_ns = h->timeout_ns;
            xa.trace = reinterpret_cast<TraceRec*>(h->trace);
            xa.trace_cap = (unsigned long long)h->trace_cap;
            e = launch_exchange(h->x_l, xa, h->stream, h->grid_cap);
        } else {
            e = launch_fused(h->x_l, h->stream, h->grid_cap);  // self messages only: no signalling
        }
        if (e) return cuda_fail("exchange kernel launch", e);
        return DDT_OK;
    }
    if (h->early) {
        cudaError_t e = cudaEventRecord(h->early_start, h->stream);
        if (e != cudaSuccess) return cuda_fail("early send: event", e);
    }
    if (h->pack_l.total_items) {
        int e = launch_fused(h->pack_l, h->stream, 0);
        if (e) return cuda_fail("pack launch", e);
    }
    bool remote = false;
    for (auto& x : h->xfers) remote |= x.peer != h->rank || h->self_nccl;
    if (remote && h->early) {
        ddt_status_t st = record_early_transfer(h);
        if (st != DDT_OK) return st;
    } else if (remote) {
        const NcclApi* n = nccl();
        if (!n) return DDT_ERR_UNSUPPORTED;
        int r = n->GroupStart();
        for (auto& x : h->xfers) {
            if ((x.peer == h->rank && !h->self_nccl) || r != 0) continue;
            if (x.send_bytes)
                r = n->Send((char*)h->send_stage + x.send_off, (size_t)x.send_bytes, kNcclUint8, x.peer, h->comm,
                            h->stream);
            if (r == 0 && x.recv_bytes)
                r = n->Recv((char*)h->recv_stage + x.recv_off, (size_t)x.recv_bytes, kNcclUint8, x.peer, h->comm,
                            h->stream);
        }
        int r2 = n->GroupEnd();
        if (r == 0) r = r2;
        if (r != 0) return nccl_fail("halo send/recv", r);
    }
    if (h->unpack_l.total_items) {
        int e = launch_fused(h->unpack_l, h->stream, 0);
        if (e) return cuda_fail("unpack launch", e);
    }
    return DDT_OK;
}

}  // namespace

extern "C" {

ddt_status_t ddt_halo_window_bytes(int32_t nrecv, const ddt_recv_t* recvs, int64_t* bytes) {
    if (nrecv < 0 || (nrecv > 0 && !recvs) || !bytes) return DDT_ERR_ARG;
    for (int i = 0; i < nrecv; i++)
        if (!recvs[i].type || recvs[i].count < 0) return DDT_ERR_ARG;
    *bytes = layout_recvs(nrecv, recvs).window_bytes;
    return DDT_OK;
}

ddt_status_t ddt_halo_create(ddt_queue_t q, const ddt_comm_t* c, int32_t nsend, const ddt_send_t* sends, int32_t nrecv,
                             const ddt_recv_t* recvs, int32_t mode, ddt_halo_t* out) {
    if (!q || !c || !out || nsend < 0 || nrecv < 0 || (nsend && !sends) || (nrecv && !recvs)) return DDT_ERR_ARG;
    if (mode != DDT_XCHG_NCCL && mode != DDT_XCHG_P2P && mode != DDT_XCHG_P2P_DIRECT && mode != DDT_XCHG_NCCL_EARLY)
        return DDT_ERR_ARG;
    const bool early = mode == DDT_XCHG_NCCL_EARLY;
    if (early) mode = DDT_XCHG_NCCL;  // the NCCL-mode plan, with per-peer early send
    const bool p2p = mode != DDT_XCHG_NCCL;
    const bool direct = mode == DDT_XCHG_P2P_DIRECT;
    if (c->nranks < 1 || c->rank < 0 || c->rank >= c->nranks) return DDT_ERR_ARG;
    if (c->nranks > 1 && !c->nccl_comm && !c->host_allgather) return DDT_ERR_ARG;  // no metadata path
    if (c->nranks > 1 && mode == DDT_XCHG_NCCL && !c->nccl_comm) return DDT_ERR_ARG;
    if (p2p && (!c->peer_windows || c->window_bytes <= 0)) return DDT_ERR_ARG;
    if (queue_sticky(q) != DDT_OK) return queue_sticky(q);
    auto* h = new (std::nothrow) ddt_halo_s();
    if (!h) return DDT_ERR_NOMEM;
    h->q = q;
    h->device = queue_device(q);
    h->stream = (cudaStream_t)queue_stream(q);
    h->rank = c->rank;
    h->nranks = c->nranks;
    h->mode = mode;
    h->early = early;
    h->comm = c->nccl_comm;
    h->ag = c->host_allgather;
    h->ag_ctx = c->host_ctx;
    DevGuard g(h->device);
    // validate messages.  Every check below is local to this rank; its status
    // is agreed (min over ranks) before the collective metadata rounds, so a
    // rank that rejects its arguments fails together with its peers instead of
    // leaving them blocked in the directory all-gather.
    ddt_status_t vst = DDT_OK;
    auto fail = [&](ddt_status_t e, const char* why) {
        if (vst == DDT_OK) {
            vst = e;
            if (why) set_error(why);
        }
    };
    std::map<std::pair<int, int>, int> seen_s, seen_r;
    for (int i = 0; i < nsend; i++) {
        auto& s = sends[i];
        if (!s.type || s.count < 0 || s.peer < 0 || s.peer >= c->nranks) {
            fail(DDT_ERR_ARG, "bad send argument");
            continue;
        }
        if (!s.type->committed) fail(DDT_ERR_STATE, "send type not committed");
        else if (s.count * s.type->size > 0 && !s.buf) fail(DDT_ERR_ARG, "null send buffer");
        if (!seen_s.emplace(std::make_pair(s.peer, s.tag), i).second) fail(DDT_ERR_ARG, "duplicate (peer, tag) send");
    }
    for (int i = 0; i < nrecv; i++) {
        auto& r = recvs[i];
        if (!r.type || r.count < 0 || r.peer < 0 || r.peer >= c->nranks) {
            fail(DDT_ERR_ARG, "bad receive argument");
            continue;
        }
        if (!r.type->committed) fail(DDT_ERR_STATE, "receive type not committed");
        else if (r.count * r.type->size > 0 && !r.buf) fail(DDT_ERR_ARG, "null receive buffer");
        else if (r.count * r.type->size > 0 && instances_overlap(r.type, r.count))
            fail(DDT_ERR_OVERLAP, "overlapping receive typemap");
        if (!seen_r.emplace(std::make_pair(r.peer, r.tag), i).second) fail(DDT_ERR_ARG, "duplicate (peer, tag) receive");
    }
    if (p2p && vst == DDT_OK) {
        // symmetric pattern of NON-EMPTY messages, required by the parity double
        // buffering / ready handshake: a rank that sends data to p must also
        // wait for data from p each exchange, or it could run two epochs ahead
        // and overwrite the window half p is still unpacking (zero-byte
        // messages produce no items and synchronise nothing)
        std::map<int, int> out_nz, in_nz;
        for (int i = 0; i < nsend; i++)
            if (sends[i].peer != c->rank && sends[i].count * sends[i].type->size > 0) out_nz[sends[i].peer]++;
        for (int i = 0; i < nrecv; i++)
            if (recvs[i].peer != c->rank && recvs[i].count * recvs[i].type->size > 0) in_nz[recvs[i].peer]++;
        for (auto& kv : out_nz)
            if (!in_nz.count(kv.first))
                fail(DDT_ERR_ARG, "P2P exchange needs a symmetric pattern (non-empty send to p => non-empty "
                                  "receive from p)");
        for (auto& kv : in_nz)
            if (!out_nz.count(kv.first))
                fail(DDT_ERR_ARG, "P2P exchange needs a symmetric pattern (non-empty receive from p => non-empty "
                                  "send to p)");
    }
    RecvLayout RL;
    if (vst == DDT_OK) {
        RL = layout_recvs(nrecv, recvs, mode == DDT_XCHG_P2P);
        if (p2p && c->window_bytes < RL.window_bytes) fail(DDT_ERR_ARG, "window smaller than ddt_halo_window_bytes()");
    }
    {
        const std::string why = vst != DDT_OK ? last_error() : "";
        ddt_status_t all = agree(h, vst);
        if (all != DDT_OK) {
            if (vst == DDT_OK) set_error("halo create failed on a peer rank");
            else set_error(why);
            delete h;  // nothing retained yet
            return all;
        }
    }
    h->sends.assign(sends, sends + nsend);
    h->recvs.assign(recvs, recvs + nrecv);
    for (auto& s : h->sends) type_retain(s.type);
    for (auto& r : h->recvs) type_retain(r.type);

    // test hook (never set in production): in P2P_DIRECT mode, route self
    // messages through the pack-free remote protocol (ready flag -> gather ->
    // scatter into the "peer's" receive buffer -> done flag), so one GPU
    // exercises and times it
    const char* svd = DDT_KNOB("DDT_SELF_VIA_DIRECT");
    const bool self_direct = direct && svd && svd[0] == '1';

    // ---- receive layout (above) and directories (receiver -> each sender)
    const int P = c->nranks;
    std::vector<std::vector<int64_t>> dir_out((size_t)P), dir_in;
    for (int p = 0; p < P; p++) {
        std::vector<int> mine;
        for (int k : RL.order)
            if (recvs[k].peer == p) mine.push_back(k);
        auto& v = dir_out[(size_t)p];
        const bool dmsg = direct && (p != c->rank || self_direct);
        v = {(int64_t)mine.size(), RL.parity_stride, RL.flags_bytes, RL.ready_off, dmsg ? 1 : 0};
        for (int k : mine) {
            v.push_back(recvs[k].tag);
            v.push_back(recvs[k].count * recvs[k].type->size);
            v.push_back(RL.data_off[(size_t)k]);
            v.push_back(RL.flag_idx[(size_t)k]);
            v.push_back(RL.lw[(size_t)k]);
            v.push_back(RL.nflags[(size_t)k]);
            v.push_back(RL.ll_ok[(size_t)k]);
            if (!dmsg) continue;
            // pack-free: publish the receive buffer (IPC handle + offset) and its layout
            int64_t words[9 + kDescWords] = {0};
            ReqDesc d;
            DeviceLayout* dl = nullptr;
            void* base = nullptr;
            cudaIpcMemHandle_t ih;
            ddt_status_t s2 = type_device_layout(recvs[k].type, h->device, &dl);
            if (s2 == DDT_OK) s2 = build_typed(recvs[k].type, dl, recvs[k].buf, recvs[k].count, &d);
            if (s2 == DDT_OK && d.kind != K_STRIDED && d.kind != K_CONTIG) {
                set_error("pack-free exchange needs closed-form (strided) receive types");
                s2 = DDT_ERR_UNSUPPORTED;
            }
            if (s2 == DDT_OK) s2 = alloc_base(recvs[k].buf, &base);
            if (s2 == DDT_OK) {
                cudaError_t e = cudaIpcGetMemHandle(&ih, base);
                if (e != cudaSuccess) s2 = cuda_fail("cudaIpcGetMemHandle(recv buffer)", e);
            }
            if (s2 != DDT_OK) {
                free_halo(h);
                return s2;
            }
            d.ptr = 0;
            std::memcpy(words, &ih, 64);
            words[8] = (int64_t)((const char*)recvs[k].buf - (const char*)base);
            std::memcpy(words + 9, &d, sizeof(ReqDesc));
            v.insert(v.end(), words, words + 9 + kDescWords);
        }
    }
    ddt_status_t st = DDT_OK;
    if (P > 1) {
        st = h->ag ? exchange_directories_host(h, dir_out, dir_in) : exchange_directories(h, dir_out, dir_in);
        if (st != DDT_OK) {
            free_halo(h);
            return st;
        }
    } else {
        dir_in.assign(1, {});
    }
    dir_in[(size_t)c->rank] = dir_out[(size_t)c->rank];
    std::vector<Directory> dirs((size_t)P);
    for (int p = 0; p < P; p++) dirs[(size_t)p] = parse_dir(dir_in[(size_t)p]);

    // ---- match sends against the peers' directories
    std::vector<const DirEntry*> match((size_t)nsend, nullptr);
    for (int i = 0; i < nsend && st == DDT_OK; i++) {
        const auto& s = sends[i];
        const Directory& d = dirs[(size_t)s.peer];
        for (auto& e : d.e)
            if (e.tag == s.tag) match[(size_t)i] = &e;
        if (!match[(size_t)i]) {
            set_error("send without a matching receive (peer " + std::to_string(s.peer) + ", tag " +
                      std::to_string(s.tag) + ")");
            st = DDT_ERR_SIZE_MISMATCH;
        } else if (match[(size_t)i]->bytes != s.count * s.type->size) {
            set_error("send/recv size mismatch (peer " + std::to_string(s.peer) + ", tag " + std::to_string(s.tag) +
                      ")");
            st = DDT_ERR_SIZE_MISMATCH;
        }
    }
    for (int p = 0; p < P && st == DDT_OK; p++) {  // every receive must have a send
        size_t nsend_p = 0;
        for (int i = 0; i < nsend; i++) nsend_p += sends[i].peer == p;
        if (nsend_p != dirs[(size_t)p].e.size()) {
            set_error("receive without a matching send");
            st = DDT_ERR_SIZE_MISMATCH;
        }
    }
    st = agree(h, st);
    if (st != DDT_OK) {
        free_halo(h);
        return st;
    }

    // test hook (never set in production): route self messages through the
    // window path instead of DirectIPC, so single-GPU tests and benchmarks
    // exercise and time the multi-GPU protocols
    const char* svw = DDT_KNOB("DDT_SELF_VIA_WINDOW");
    const bool self_window = p2p && !direct && svw && svw[0] == '1';
    auto remote = [&](int peer) { return peer != c->rank || self_window || self_direct; };
    // the same for NCCL mode (needs an NCCL communicator, e.g. a 1-rank one):
    // self messages go pack -> staging -> ncclSend/ncclRecv to self -> unpack
    const char* svn = DDT_KNOB("DDT_SELF_VIA_NCCL");
    h->self_nccl = mode == DDT_XCHG_NCCL && c->nccl_comm && svn && svn[0] == '1';
    auto remote_n = [&](int peer) { return peer != c->rank || h->self_nccl; };

    // ---- second metadata round (window mode): sender -> receiver, which
    // messages travel in the LL format (receiver offered it, sender can do 8-B)
    std::map<std::pair<int, int>, int> send_ll, recv_ll;
    if (p2p && !direct) {
        std::vector<std::vector<int64_t>> out2((size_t)P), in2;
        std::vector<std::vector<std::pair<int64_t, int64_t>>> lists((size_t)P);
        for (int i = 0; i < nsend; i++) {
            const auto& s = sends[i];
            if (s.count * s.type->size == 0 || !remote(s.peer)) continue;
            const int lw_s = std::min(4, side_lw(s.type, s.buf, s.count));
            const char* nl = DDT_KNOB("DDT_NO_LL");  // experiments: flag protocol only
            const int ll = (match[(size_t)i]->ll_ok && lw_s >= 3 && !(nl && nl[0] == '1')) ? 1 : 0;
            send_ll[{s.peer, s.tag}] = ll;
            lists[(size_t)s.peer].push_back({s.tag, ll});
        }
        for (int p = 0; p < P; p++) {
            std::sort(lists[(size_t)p].begin(), lists[(size_t)p].end());
            out2[(size_t)p].push_back((int64_t)lists[(size_t)p].size());
            for (auto& e : lists[(size_t)p]) {
                out2[(size_t)p].push_back(e.first);
                out2[(size_t)p].push_back(e.second);
            }
        }
        if (P > 1) {
            st = h->ag ? exchange_directories_host(h, out2, in2) : exchange_directories(h, out2, in2);
            if (st != DDT_OK) {
                free_halo(h);
                return st;
            }
        } else {
            in2.assign(1, {});
        }
        in2[(size_t)c->rank] = out2[(size_t)c->rank];
        for (int p = 0; p < P; p++) {
            const auto& v = in2[(size_t)p];
            for (int64_t k = 0; v.size() >= 1 && k < v[0] && (size_t)(2 + 2 * k) < v.size() + 1; k++)
                recv_ll[{p, (int)v[(size_t)(1 + 2 * k)]}] = (int)v[(size_t)(2 + 2 * k)];
        }
    }

    // ---- build the device work tables
    // pack: typed send buffer -> packed slot; unpack: packed slot -> typed recv buffer
    auto add_req = [&](HostBatch& b, ddt_type_s* t, int op, const void* src, const void* dst, int64_t count,
                       int* lw) -> ddt_status_t {
        DeviceLayout* dl = nullptr;
        ddt_status_t s2 = type_device_layout(t, h->device, &dl);
        ReqDesc sd, dd;
        if (s2 == DDT_OK) s2 = build_request(op, t, dl, src, dst, count, &sd, &dd);
        if (s2 != DDT_OK) return s2;
        b.add(sd, dd);
        if (lw) *lw = sd.lw;
        return DDT_OK;
    };
    // Self messages never touch a staging buffer or window: one DirectIPC
    // descriptor gathers the send layout and scatters straight into the
    // matching receive layout -- 2S instead of 4S HBM bytes.
    auto self_recv = [&](int tag) {
        for (int i = 0; i < nrecv; i++)
            if (recvs[i].peer == c->rank && recvs[i].tag == tag) return i;
        return -1;
    };
    auto add_direct = [&](HostBatch& b, const ddt_send_t& s, const ddt_recv_t& r, bool with_x) -> ddt_status_t {
        DeviceLayout *dls = nullptr, *dld = nullptr;
        ddt_status_t s2 = type_device_layout(s.type, h->device, &dls);
        if (s2 == DDT_OK) s2 = type_device_layout(r.type, h->device, &dld);
        ReqDesc d, a;
        if (s2 == DDT_OK) s2 = build_direct(s.type, dls, s.buf, s.count, r.type, dld, r.buf, r.count, &d, &a);
        if (s2 != DDT_OK) return s2;
        b.add(d, a);
        if (with_x) b.xinfo.push_back(XInfo{});
        return DDT_OK;
    };
    for (auto& s : h->sends) h->bytes += s.count * s.type->size;
    if (mode == DDT_XCHG_NCCL) {
        cudaError_t e = cudaMalloc(&h->recv_stage, (size_t)RL.parity_stride);
        // send staging: one region per remote peer reproducing the receiver's layout
        std::map<int, std::pair<int64_t, int64_t>> span;  // peer -> (first_off, end_off) in the peer's layout
        for (int i = 0; i < nsend; i++) {
            if (!remote_n(sends[i].peer)) continue;
            int64_t a = match[(size_t)i]->data_off, b = a + match[(size_t)i]->bytes;
            auto it = span.find(sends[i].peer);
            if (it == span.end()) span[sends[i].peer] = {a, b};
            else it->second = {std::min(it->second.first, a), std::max(it->second.second, b)};
        }
        std::map<int, int64_t> region;
        int64_t soff = 0;
        for (auto& kv : span) {
            region[kv.first] = soff;
            soff = round_up(soff + (kv.second.second - kv.second.first), 256);
        }
        if (e == cudaSuccess) e = cudaMalloc(&h->send_stage, (size_t)std::max<int64_t>(soff, 256));
        if (e != cudaSuccess) {
            free_halo(h);
            return cuda_fail("cudaMalloc(staging)", e);
        }
        // my receive spans per remote peer
        std::map<int, std::pair<int64_t, int64_t>> rspan;
        for (int i = 0; i < nrecv; i++) {
            if (!remote_n(recvs[i].peer)) continue;
            int64_t a = RL.data_off[(size_t)i], b = a + recvs[i].count * recvs[i].type->size;
            auto it = rspan.find(recvs[i].peer);
            if (it == rspan.end()) rspan[recvs[i].peer] = {a, b};
            else it->second = {std::min(it->second.first, a), std::max(it->second.second, b)};
        }
        std::map<int, Xfer> xf;
        for (auto& kv : span) {
            Xfer& x = xf[kv.first];
            x.peer = kv.first;
            x.send_off = region[kv.first];
            x.send_bytes = kv.second.second - kv.second.first;
        }
        for (auto& kv : rspan) {
            Xfer& x = xf[kv.first];
            x.peer = kv.first;
            x.recv_off = kv.second.first;
            x.recv_bytes = kv.second.second - kv.second.first;
        }
        for (auto& kv : xf) h->xfers.push_back(kv.second);
        HostBatch packb, unpackb;
        // remote packs first, peer by peer (early send: the first peers' data is
        // ready first), then the self messages
        std::vector<int> sorder((size_t)nsend);
        for (int i = 0; i < nsend; i++) sorder[(size_t)i] = i;
        std::stable_sort(sorder.begin(), sorder.end(), [&](int a, int b) {
            const bool ra = remote_n(sends[a].peer), rb = remote_n(sends[b].peer);
            if (ra != rb) return ra;
            return ra && sends[a].peer < sends[b].peer;
        });
        std::map<int, std::vector<int>> peer_ctr;  // early send: remote peer -> its counters
        int nctr = 0;
        for (int i : sorder) {
            if (st != DDT_OK) break;
            const auto& s = sends[i];
            if (s.count * s.type->size == 0) continue;
            if (!remote_n(s.peer)) {
                st = add_direct(packb, s, recvs[self_recv(s.tag)], false);
                continue;
            }
            char* dst = (char*)h->send_stage + region[s.peer] + (match[(size_t)i]->data_off - span[s.peer].first);
            st = add_req(packb, s.type, OP_PACK, s.buf, dst, s.count, nullptr);
            if (st == DDT_OK && early) peer_ctr[s.peer].push_back(nctr++);
        }
        if (st == DDT_OK && early) {
            // completion counters (device): the CTA finishing a remote pack
            // request's last item increments its counter (fused_kernel.cu)
            if (!memops()) {
                set_error("NCCL_EARLY needs stream memory operations (cuStreamWaitValue32)");
                st = DDT_ERR_UNSUPPORTED;
            }
            const size_t nb = sizeof(uint32_t) * (size_t)std::max(nctr, 1);
            cudaError_t e = st == DDT_OK ? cudaMalloc((void**)&h->early_ctr, nb) : cudaSuccess;
            if (e == cudaSuccess && st == DDT_OK) e = cudaMalloc((void**)&h->early_done, nb);
            if (e == cudaSuccess && st == DDT_OK) e = cudaMemset(h->early_ctr, 0, nb);
            if (e == cudaSuccess && st == DDT_OK) e = cudaMemset(h->early_done, 0, nb);
            if (e == cudaSuccess && st == DDT_OK) e = cudaEventCreateWithFlags(&h->early_start, cudaEventDisableTiming);
            if (e != cudaSuccess) st = cuda_fail("early send setup", e);
            int k = 0;
            for (size_t r = 0; r < packb.descs.size() && st == DDT_OK; r++) {
                ReqDesc& d = packb.descs[r];
                if (d.op != OP_PACK) continue;  // remote packs come first, in counter order
                d.resp = (uint64_t)(uintptr_t)(h->early_ctr + k);
                d.resp_val = kRespIncrement;
                d.done_ctr = (uint64_t)(uintptr_t)(h->early_done + k);
                k++;
            }
            for (size_t xi = 0; xi < h->xfers.size() && st == DDT_OK; xi++) {
                const Xfer& x = h->xfers[xi];
                if (!remote_n(x.peer)) continue;
                ddt_halo_s::EarlyPeer P;
                P.xfer = xi;
                auto it = peer_ctr.find(x.peer);
                if (it != peer_ctr.end()) P.ctr = it->second;
                e = cudaStreamCreateWithFlags(&P.s, cudaStreamNonBlocking);
                if (e == cudaSuccess) e = cudaEventCreateWithFlags(&P.done, cudaEventDisableTiming);
                h->epeers.push_back(P);
                if (e != cudaSuccess) st = cuda_fail("early send streams", e);
            }
            std::sort(h->epeers.begin(), h->epeers.end(), [&](const ddt_halo_s::EarlyPeer& a,
                                                              const ddt_halo_s::EarlyPeer& b) {
                return h->xfers[a.xfer].peer < h->xfers[b.xfer].peer;
            });
        }
        for (int i = 0; i < nrecv && st == DDT_OK; i++) {
            const auto& r = recvs[i];
            if (r.count * r.type->size == 0 || !remote_n(r.peer)) continue;
            st = add_req(unpackb, r.type, OP_UNPACK, (char*)h->recv_stage + RL.data_off[(size_t)i], r.buf, r.count,
                         nullptr);
        }
        packb.ticket = unpackb.ticket = queue_ticket(q);
        if (st == DDT_OK && !packb.descs.empty()) st = make_table(packb, h->pack_l, queue_sm_count(q));
        if (st == DDT_OK && !unpackb.descs.empty()) st = make_table(unpackb, h->unpack_l, queue_sm_count(q));
        h->launches = (packb.descs.empty() ? 0 : 1) + (unpackb.descs.empty() ? 0 : 1);
    } else {
        // P2P: one kernel.  Item order = deadlock-freedom order (fused_kernel.cu):
        // items that never wait first (ready signals, remote packs, self directs),
        // then pack-free remote directs (wait for the peer's ready flag), then the
        // items that wait for data (unpacks / completion waits).
        HostBatch xb;
        char* mywin = (char*)c->peer_windows[c->rank];
        uint32_t npack = 0;
        ReqDesc none;
        std::memset(&none, 0, sizeof(none));
        none.kind = K_CONTIG;
        none.op = OP_SIGNAL;
        std::vector<int> rpeers;  // remote peers we receive from (== send to: symmetric)
        for (int i = 0; i < nrecv; i++)
            if (remote(recvs[i].peer) && recvs[i].count * recvs[i].type->size > 0) rpeers.push_back(recvs[i].peer);
        std::sort(rpeers.begin(), rpeers.end());
        rpeers.erase(std::unique(rpeers.begin(), rpeers.end()), rpeers.end());
        if (direct) {  // "ready": this rank entered the exchange, its ghosts may be overwritten
            for (int p : rpeers) {
                XInfo x{};
                x.signal = (uint64_t)(uintptr_t)((char*)c->peer_windows[p] + dirs[(size_t)p].ready_base + 8 * c->rank);
                x.nitems = 1;
                x.fanout = 1;
                const char* fs0 = DDT_KNOB("DDT_FORCE_SYS_SCOPE");  // experiments: emulate a peer GPU's flags
                x.gpu_scope = (p == c->rank && !(fs0 && fs0[0] == '1')) ? 1u : 0u;  // self (test hook)
                xb.add(none, none);
                xb.xinfo.push_back(x);
            }
        }
        for (int i = 0; i < nsend && st == DDT_OK && !direct; i++) {
            const auto& s = sends[i];
            if (s.count * s.type->size == 0 || !remote(s.peer)) continue;
            const Directory& d = dirs[(size_t)s.peer];
            char* win = (char*)c->peer_windows[s.peer];
            if (send_ll[{s.peer, s.tag}]) {  // LL: the data carries its own epoch, no signal
                DeviceLayout* dl = nullptr;
                ReqDesc sd, dd;
                st = type_device_layout(s.type, h->device, &dl);
                if (st == DDT_OK)
                    st = build_ll(OP_PACK, s.type, dl, s.buf, win + d.data_base + match[(size_t)i]->data_off, s.count,
                                  &sd, &dd);
                if (st != DDT_OK) break;
                sd.xub = (uint8_t)xub_for(s.count * s.type->size);  // no flags: free to pick the item size
                xb.add(sd, dd);
                XInfo x{};
                x.parity_stride = d.parity_stride;
                xb.xinfo.push_back(x);
                continue;
            }
            int lw = 0;
            st = add_req(xb, s.type, OP_PACK, s.buf, win + d.data_base + match[(size_t)i]->data_off, s.count, &lw);
            if (st == DDT_OK) xb.descs.back().xub = (uint8_t)xub_for(s.count * s.type->size);
            XInfo x{};
            x.signal = (uint64_t)(uintptr_t)(win + 8 * match[(size_t)i]->flag_idx);
            x.counter = npack++;
            x.parity_stride = d.parity_stride;
            // same vector width on both sides => identical chunking: per-chunk flags
            // (DDT_CHUNK_FLAGS=0: experiments, release every flag at message end)
            const char* cf = DDT_KNOB("DDT_CHUNK_FLAGS");
            x.per_item = (lw == match[(size_t)i]->lw && !(cf && cf[0] == '0')) ? 1u : 0u;
            // the reader of this flag runs on our own device (self window): gpu scope suffices
            const char* fs = DDT_KNOB("DDT_FORCE_SYS_SCOPE");  // experiments: emulate a peer GPU's flags
            x.gpu_scope = (s.peer == c->rank && !(fs && fs[0] == '1')) ? 1u : 0u;
            x.fanout = (uint32_t)match[(size_t)i]->nflags;  // else: all of the receiver's flags at the end
            xb.xinfo.push_back(x);
        }
        for (int i = 0; i < nsend && st == DDT_OK; i++) {
            const auto& s = sends[i];
            if (s.count * s.type->size == 0 || remote(s.peer)) continue;
            st = add_direct(xb, s, recvs[self_recv(s.tag)], true);
        }
        for (int i = 0; i < nsend && st == DDT_OK && direct; i++) {
            const auto& s = sends[i];
            if (s.count * s.type->size == 0 || !remote(s.peer)) continue;
            const DirEntry& e = *match[(size_t)i];
            ReqDesc sd, dd = e.desc;
            if (s.peer == c->rank) {  // self through the remote protocol (test hook): no IPC mapping needed
                dd.ptr = (uint64_t)(uintptr_t)recvs[self_recv(s.tag)].buf;
            } else {
                cudaIpcMemHandle_t ih;
                std::memcpy(&ih, e.ipc, 64);
                void* mapped = nullptr;
                cudaError_t ce = cudaIpcOpenMemHandle(&mapped, ih, cudaIpcMemLazyEnablePeerAccess);
                if (ce != cudaSuccess) {
                    st = cuda_fail("cudaIpcOpenMemHandle(peer recv buffer)", ce);
                    break;
                }
                h->ipc_opened.push_back(mapped);
                dd.ptr = (uint64_t)(uintptr_t)((char*)mapped + e.alloc_off);
            }
            DeviceLayout* dl = nullptr;
            st = type_device_layout(s.type, h->device, &dl);
            if (st == DDT_OK) st = build_typed(s.type, dl, s.buf, s.count, &sd);
            const int lw = std::min<int>(sd.lw, dd.lw);
            if (st == DDT_OK && sd.lw != lw) st = rescale_desc(&sd, lw);
            if (st == DDT_OK && dd.lw != lw) st = rescale_desc(&dd, lw);
            if (st == DDT_OK && sd.nvec != dd.nvec) st = DDT_ERR_SIZE_MISMATCH;
            if (st != DDT_OK) break;
            sd.op = dd.op = OP_DIRECT;
            sd.xub = (uint8_t)xub_for(s.count * s.type->size);  // one done flag per message: any chunking
            xb.add(sd, dd);
            XInfo x{};
            x.signal = (uint64_t)(uintptr_t)((char*)c->peer_windows[s.peer] + 8 * e.flag_idx);
            x.wait = (uint64_t)(uintptr_t)(mywin + RL.ready_off + 8 * s.peer);
            x.counter = npack++;
            x.fanout = 1;
            const char* fs1 = DDT_KNOB("DDT_FORCE_SYS_SCOPE");
            x.gpu_scope = (s.peer == c->rank && !(fs1 && fs1[0] == '1')) ? 1u : 0u;  // self (test hook)
            xb.xinfo.push_back(x);
        }
        for (int i = 0; i < nrecv && st == DDT_OK; i++) {
            const auto& r = recvs[i];
            if (r.count * r.type->size == 0 || !remote(r.peer)) continue;
            XInfo x{};
            x.wait = (uint64_t)(uintptr_t)(mywin + 8 * RL.flag_idx[(size_t)i]);
            if (direct) {  // the data lands by itself; wait for its completion flag
                xb.add(none, none);
            } else if (recv_ll[{r.peer, r.tag}]) {  // LL: every 8 B validates itself
                DeviceLayout* dl = nullptr;
                ReqDesc sd, dd;
                st = type_device_layout(r.type, h->device, &dl);
                if (st == DDT_OK)
                    st = build_ll(OP_UNPACK, r.type, dl, r.buf, mywin + RL.flags_bytes + RL.data_off[(size_t)i],
                                  r.count, &sd, &dd);
                if (st != DDT_OK) break;
                sd.xub = (uint8_t)xub_for(r.count * r.type->size);
                xb.add(sd, dd);
                x.wait = 0;
                x.parity_stride = RL.parity_stride;
            } else {  // unpack chunk k as soon as the sender's chunk k has landed
                st = add_req(xb, r.type, OP_UNPACK, mywin + RL.flags_bytes + RL.data_off[(size_t)i], r.buf, r.count,
                             nullptr);
                if (st == DDT_OK) xb.descs.back().xub = (uint8_t)xub_for(r.count * r.type->size);
                x.parity_stride = RL.parity_stride;
                x.per_item = 1;
            }
            const char* fs2 = DDT_KNOB("DDT_FORCE_SYS_SCOPE");
            x.gpu_scope = (r.peer == c->rank && !(fs2 && fs2[0] == '1')) ? 1u : 0u;  // the writer runs on this GPU
            xb.xinfo.push_back(x);
        }
        for (const auto& x : xb.xinfo) h->x_flags |= x.signal != 0 || x.wait != 0;
        for (size_t i = 0; i < xb.descs.size(); i++)  // LL windows need the exchange kernel (and its epoch)
            h->x_flags |= xb.descs[i].kind == K_LL || xb.aux[xb.descs[i].aux].kind == K_LL;
        // control block (item tick -> epoch, message counters) first: the
        // table carries the tick's address
        size_t ctrl_bytes = sizeof(XCtrl) + sizeof(unsigned long long) * std::max<size_t>(npack, 1);
        if (st == DDT_OK) {
            cudaError_t e = cudaMalloc(&h->ctrl, ctrl_bytes);
            if (e == cudaSuccess) e = cudaMemset(h->ctrl, 0, ctrl_bytes);
            if (e == cudaSuccess) e = cudaHostAlloc((void**)&h->err_host, sizeof(int), cudaHostAllocMapped);
            if (e == cudaSuccess) {
                *h->err_host = 0;
                e = cudaHostGetDevicePointer((void**)&h->err_dev, h->err_host, 0);
            }
            if (e != cudaSuccess) st = cuda_fail("exchange control block", e);
        }
        if (st == DDT_OK && !xb.descs.empty()) {
            // exchange plans chunk every message alike on both sides (kXchgUb)
            for (size_t i = 0; i < xb.descs.size(); i++)
                if (xb.xinfo[i].signal) xb.xinfo[i].nitems = desc_items(xb.descs[i], kXchgUb);
            // exchange kernels claim items from the plan's own ticket (item
            // order = claim order: deadlock freedom without co-residency);
            // flag-free plans (self messages only) run the plain fused kernel
            // with the queue's ticket and an adaptive item size
            xb.ticket = h->x_flags ? (uint64_t)(uintptr_t)((char*)h->ctrl + offsetof(XCtrl, tick))
                                   : queue_ticket(q);
            st = make_table(xb, h->x_l, queue_sm_count(q), h->x_flags ? kXchgUb : 0);
        }
        h->launches = xb.descs.empty() ? 0 : 1;
    }
    if (st == DDT_OK) {
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) st = cuda_fail("halo create", e);
    }
    if (st != DDT_OK) {
        free_halo(h);
        return st;
    }
    *out = h;
    return DDT_OK;
}

ddt_status_t ddt_halo_set_timeout(ddt_halo_t h, int64_t timeout_ns) {
    if (!h || timeout_ns <= 0) return DDT_ERR_ARG;
    h->timeout_ns = (uint64_t)timeout_ns;
    if (h->gexec) {  // the old value is baked into the captured launch
        cudaGraphExecDestroy(h->gexec);
        h->gexec = nullptr;
    }
    return DDT_OK;
}

ddt_status_t ddt_halo_set_trace(ddt_halo_t h, void* dev_records, int64_t capacity) {
    if (!h || capacity < 0 || (capacity > 0 && !dev_records)) return DDT_ERR_ARG;
    if (!h->ctrl) return DDT_ERR_STATE;  // tracing covers the fused exchange kernel (P2P plans)
    DevGuard g(h->device);
    h->trace = capacity > 0 ? dev_records : nullptr;
    h->trace_cap = capacity;
    unsigned int zero = 0;
    cudaError_t e =
        cudaMemcpyAsync((char*)h->ctrl + offsetof(XCtrl, trace_n), &zero, 4, cudaMemcpyHostToDevice, h->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
    return e == cudaSuccess ? DDT_OK : cuda_fail("halo trace", e);
}

ddt_status_t ddt_halo_set_graph(ddt_halo_t h, int32_t use_graph) {
    if (!h) return DDT_ERR_ARG;
    h->use_graph = use_graph != 0;
    return DDT_OK;
}

ddt_status_t ddt_exchange(ddt_halo_t h) {
    if (!h) return DDT_ERR_ARG;
    ddt_status_t st = queue_sticky(h->q);
    if (st != DDT_OK) return st;
    if (h->err_host && *(volatile int*)h->err_host) {
        set_error("P2P exchange: a peer flag wait exceeded the timeout");
        queue_set_sticky(h->q, DDT_ERR_TIMEOUT);
        return DDT_ERR_TIMEOUT;
    }
    DevGuard g(h->device);
    // every plan may be captured (the P2P epoch is device-resident) and, with
    // ddt_halo_set_graph, replays its own captured graph
    if (h->use_graph && h->stream) {
        if (!h->gexec) {
            cudaError_t e = cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal);
            if (e != cudaSuccess) return cuda_fail("graph capture begin", e);
            ddt_status_t rs = record_exchange(h);
            cudaGraph_t graph = nullptr;
            e = cudaStreamEndCapture(h->stream, &graph);
            if (rs != DDT_OK) {
                if (graph) cudaGraphDestroy(graph);
                return rs;
            }
            if (e != cudaSuccess) return cuda_fail("graph capture end", e);
            e = cudaGraphInstantiate(&h->gexec, graph, 0);
            cudaGraphDestroy(graph);
            if (e != cudaSuccess) return cuda_fail("graph instantiate", e);
        }
        cudaError_t e = cudaGraphLaunch(h->gexec, h->stream);
        if (e != cudaSuccess) return cuda_fail("graph launch", e);
    } else {
        st = record_exchange(h);
        if (st != DDT_OK) {
            queue_set_sticky(h->q, st);
            return st;
        }
    }
    queue_count_launches(h->q, h->launches, 2 * h->bytes);
    return DDT_OK;
}

ddt_status_t ddt_halo_launches_per_exchange(ddt_halo_t h, int32_t* launches) {
    if (!h || !launches) return DDT_ERR_ARG;
    *launches = h->launches;
    return DDT_OK;
}

ddt_status_t ddt_halo_destroy(ddt_halo_t h) {
    if (!h) return DDT_ERR_ARG;
    {
        DevGuard g(h->device);
        if (h->stream) cudaStreamSynchronize(h->stream);
        else cudaDeviceSynchronize();
        free_halo(h);
    }
    return DDT_OK;
}

}  // extern "C"
