// batch.cpp -- the work table in its two launch forms.
//
// The paper hands the fused kernel "an array of requests" (§IV-A.2) and
// partitions thread blocks over requests by size (§IV-A.3).  Here the
// partition is an exclusive prefix sum of per-request item counts
// (kItemVecs vectors per item); the kernel maps item -> request by binary
// search.  Batches of up to kParamLarge requests travel inside the kernel's
// parameters, so ddt_flush is exactly one stream operation; larger batches are
// serialised into a device table (one cudaMemcpyAsync per flush, or once for
// persistent plans and halo plans).
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "ddt_internal.h"

namespace ddt {

// Exclusive prefix of item counts; a group of m members occupies m * n items
// and every member's entry holds the group's first item (device_desc.h).
static uint32_t fill_prefix(uint32_t* prefix, const HostBatch& b, int ub) {
    const std::vector<ReqDesc>& d = b.descs;
    uint64_t acc = 0;
    for (size_t i = 0; i < d.size();) {
        const size_t m = b.gm.empty() ? 1 : std::max<uint32_t>(1, b.gm[i]);
        for (size_t j = 0; j < m; j++) prefix[i + j] = (uint32_t)acc;
        // the second member of an exchange pair runs inside its partner's items
        // (zero items: the kernel's "largest r with prefix[r] <= item" search
        // never lands on it)
        const bool partner = b.order.empty() && i > 0 && d[i - 1].pair;
        acc += partner ? 0u : (uint64_t)m * desc_items(d[i], ub);
        i += m;
    }
    prefix[d.size()] = (uint32_t)acc;
    return (uint32_t)acc;
}

static size_t pad16(size_t v) { return (v + 15) & ~(size_t)15; }

// Item order (experiments: DDT_ITEM_ORDER=blocked); cyclic is the default.
static uint32_t batch_flags(const HostBatch& b) {
    const char* e = DDT_KNOB("DDT_ITEM_ORDER");
    uint32_t f = (e && e[0] == 'b') ? kBatchBlocked : 0u;
    if (!b.gm.empty()) f |= kBatchGrouped;
    return f;
}

// An LL unpack spins on its window data: it waits like a flagged unpack.
static int exchange_class(const HostBatch& b, size_t i) {
    if (b.xinfo.empty()) return 0;
    const bool waits = b.xinfo[i].wait != 0 || b.descs[i].kind == K_LL;
    return (waits ? 2 : 0) | (b.xinfo[i].signal ? 1 : 0);
}

void group_equal_requests(HostBatch& b, int ub, int max_m) {
    const char* off = DDT_KNOB("DDT_NO_GROUP");  // experiments: no interleaving
    const size_t n = b.descs.size();
    if ((off && off[0] == '1') || n < 2 || max_m < 2) return;
    std::vector<size_t> order;
    std::vector<uint32_t> gm;
    order.reserve(n);
    for (size_t lo = 0; lo < n;) {
        size_t hi = lo + 1;
        while (hi < n && exchange_class(b, hi) == exchange_class(b, lo)) hi++;
        // within [lo, hi): requests with equal item counts, in first-seen order
        std::vector<bool> taken(hi - lo, false);
        for (size_t i = lo; i < hi; i++) {
            if (taken[i - lo]) continue;
            const uint32_t it = desc_items(b.descs[i], ub);
            std::vector<size_t> g{i};
            taken[i - lo] = true;
            for (size_t j = i + 1; j < hi && it > 0 && g.size() < (size_t)max_m; j++)
                if (!taken[j - lo] && desc_items(b.descs[j], ub) == it) {
                    g.push_back(j);
                    taken[j - lo] = true;
                }
            for (size_t k : g) {
                order.push_back(k);
                gm.push_back((uint32_t)g.size());
            }
        }
        lo = hi;
    }
    bool any = false;
    for (uint32_t m : gm) any |= m > 1;
    if (!any) return;
    HostBatch out;
    out.ticket = b.ticket;
    for (size_t k : order) {
        out.add(b.descs[k], b.aux[b.descs[k].aux]);
        if (!b.xinfo.empty()) out.xinfo.push_back(b.xinfo[k]);
    }
    out.gm = std::move(gm);
    b = std::move(out);
}

// Segment length (bytes) and phase (start address mod 16) of one closed-form
// side at 8-B vectors; false if its segments do not all share one phase.
// L = 0: contiguous side, segment length free (the other side's).
static bool side_phase(const ReqDesc& d, uint64_t total, uint64_t& L, int& phase) {
    if (d.kind == K_CONTIG) {
        L = 0;
        phase = (int)(d.ptr & 15);
        return true;
    }
    L = (uint64_t)d.vps.d << 3;
    if (L == 0 || total % L) return false;
    phase = (int)((d.ptr + (uint64_t)d.base) & 15);
    if (total / L > 1) {
        for (int k = 0; k < d.ndim; k++)
            if (d.stride[k] & 15) return false;
        if (d.extent & 15) return false;
    }
    return true;
}

static bool try_phase(ReqDesc& S, ReqDesc& D) {
    if (S.ph || D.ph || S.lw != 3 || D.lw != 3 || S.nvec == 0 || S.nvec != D.nvec) return false;
    for (const ReqDesc* d : {&S, &D})
        if (d->kind != K_STRIDED && d->kind != K_CONTIG) return false;
    const uint64_t total = (uint64_t)S.nvec << 3;
    uint64_t Ls, Ld;
    int ps, pd;
    if (!side_phase(S, total, Ls, ps) || !side_phase(D, total, Ld, pd) || ps != pd || (ps & 7)) return false;
    if (Ls && Ld && Ls != Ld) return false;
    const uint64_t L = Ls ? Ls : (Ld ? Ld : total);
    const uint64_t nseg = total / L;
    if (nseg > 1 && (L & 15) && (S.kind == K_CONTIG || D.kind == K_CONTIG)) return false;  // phase would flip
    const uint64_t hd = ps == 8, tl = ((ps + L) & 15) == 8;
    const uint64_t m = (L - 8 * hd - 8 * tl) / 16;
    if (m < 2) return false;
    const uint64_t U = hd + m + tl;
    if (nseg * U >= (1ull << 32)) return false;
    for (ReqDesc* d : {&S, &D}) {
        d->ph = (uint8_t)(kPhOn | (hd ? kPhHead : 0) | (tl ? kPhTail : 0));
        d->lw = 4;
        d->vps = make_div((uint32_t)U);
        d->nvec = (uint32_t)(nseg * U);
    }
    return true;
}

void phase_batch(HostBatch& b) {
    const char* off = DDT_KNOB("DDT_NO_PHASE");  // experiments: plain 8-B vectors
    if (off && off[0] == '1') return;
    for (const auto* v : {&b.descs, &b.aux})
        for (const ReqDesc& d : *v)
            if (d.nvec && d.kind != K_STRIDED && d.kind != K_CONTIG && d.kind != K_LL) return;
    for (size_t i = 0; i < b.descs.size(); i++) {
        if (!b.xinfo.empty() && (b.xinfo[i].signal || b.xinfo[i].wait)) continue;
        ReqDesc& S = b.descs[i];
        if (S.op == OP_SIGNAL) continue;
        try_phase(S, b.aux[S.aux]);
    }
}

// Two closed-form sides walk the same lattice of segments with bases less
// than one innermost stride apart (same rows).
static bool same_lattice(const ReqDesc& a, const ReqDesc& c) {
    if (a.kind != K_STRIDED || c.kind != K_STRIDED || a.ndim != c.ndim || a.ndim == 0 || a.lw != c.lw ||
        a.vps.d != c.vps.d || a.extent != c.extent || a.ph || c.ph)
        return false;
    for (int k = 0; k < a.ndim; k++)
        if (a.radix[k].d != c.radix[k].d || a.stride[k] != c.stride[k]) return false;
    const int64_t pa = (int64_t)a.ptr + a.base, pc = (int64_t)c.ptr + c.base;
    const int64_t d = pa > pc ? pa - pc : pc - pa;
    return d < (a.stride[0] < 0 ? -a.stride[0] : a.stride[0]);
}

// Pair requests whose both sides walk the same short-segment lattice (see
// device_desc.h kSpreadShift): partners become adjacent, the first carries
// pair = 1.  Spread (non-exchange, plain) batches only.  DDT_NO_PAIR=1: off.
void pair_requests(HostBatch& b) {
    const char* off = DDT_KNOB("DDT_NO_PAIR");
    if ((off && off[0] == '1') || !b.gm.empty()) return;
    const size_t n = b.descs.size();
    std::vector<int> partner(n, -1);
    bool any = false;
    for (size_t i = 0; i < n; i++) {
        const ReqDesc& A = b.descs[i];
        if (partner[i] >= 0 || A.resp || !(A.l2_64 || b.aux[A.aux].l2_64) || A.nvec == 0) continue;
        for (size_t j = i + 1; j < n; j++) {
            const ReqDesc& B = b.descs[j];
            if (partner[j] >= 0 || B.resp || B.nvec != A.nvec || B.op != A.op) continue;
            if (!same_lattice(A, B) || !same_lattice(b.aux[A.aux], b.aux[B.aux])) continue;
            partner[i] = (int)j;
            partner[j] = (int)i;
            any = true;
            break;
        }
    }
    if (!any) return;
    HostBatch out;
    out.ticket = b.ticket;
    for (size_t i = 0; i < n; i++) {
        if (partner[i] >= 0 && (size_t)partner[i] < i) continue;  // placed with its partner
        ReqDesc d = b.descs[i];
        d.pair = partner[i] >= 0 ? 1 : 0;
        out.add(d, b.aux[b.descs[i].aux]);
        if (!b.xinfo.empty()) out.xinfo.push_back(b.xinfo[i]);
        if (partner[i] >= 0) {
            out.add(b.descs[(size_t)partner[i]], b.aux[b.descs[(size_t)partner[i]].aux]);
            if (!b.xinfo.empty()) out.xinfo.push_back(b.xinfo[(size_t)partner[i]]);
        }
    }
    b = std::move(out);
}

// Exchange pairs (fused_kernel.cu run_pair_x): two requests of an exchange
// batch, both non-waiting or both waiting, neither a remote direct nor a
// signal-only item, with equal vector counts and item sizes, whose typed sides
// walk the same short-segment lattice and whose packed sides are both windows
// of one kind (K_CONTIG or K_LL).  Partners become adjacent (relative order of
// the waiting / non-waiting partition kept).  DDT_NO_XPAIR=1: off.
bool pair_exchange_requests(HostBatch& b) {
    const char* off = DDT_KNOB("DDT_NO_XPAIR");
    if ((off && off[0] == '1') || !b.gm.empty() || b.xinfo.size() != b.descs.size()) return false;
    const size_t n = b.descs.size();
    auto waits = [&](size_t i) { return b.xinfo[i].wait != 0 || b.descs[i].kind == K_LL; };
    auto typed = [&](size_t i) -> const ReqDesc& {
        return b.descs[i].op == OP_PACK ? b.descs[i] : b.aux[b.descs[i].aux];
    };
    auto packed = [&](size_t i) -> const ReqDesc& {
        return b.descs[i].op == OP_PACK ? b.aux[b.descs[i].aux] : b.descs[i];
    };
    std::vector<int> partner(n, -1);
    bool any = false;
    for (size_t i = 0; i < n; i++) {
        const ReqDesc& A = b.descs[i];
        if (partner[i] >= 0 || A.resp || A.nvec == 0 || (A.op != OP_PACK && A.op != OP_UNPACK)) continue;
        if (b.xinfo[i].wait && b.xinfo[i].signal) continue;  // remote directs
        if (!typed(i).l2_64) continue;                        // short segments only (x faces)
        for (size_t j = i + 1; j < n; j++) {
            const ReqDesc& B = b.descs[j];
            if (partner[j] >= 0 || B.resp || B.nvec != A.nvec || B.op != A.op || B.xub != A.xub) continue;
            if (waits(i) != waits(j) || (b.xinfo[j].wait && b.xinfo[j].signal)) continue;
            const ReqDesc &pa = packed(i), &pb = packed(j);
            if (pa.kind != pb.kind || (pa.kind != K_CONTIG && pa.kind != K_LL) || pa.lw != pb.lw) continue;
            if (!same_lattice(typed(i), typed(j))) continue;
            partner[i] = (int)j;
            partner[j] = (int)i;
            any = true;
            break;
        }
    }
    if (!any) return false;
    HostBatch out;
    out.ticket = b.ticket;
    for (size_t i = 0; i < n; i++) {
        if (partner[i] >= 0 && (size_t)partner[i] < i) continue;  // placed with its partner
        ReqDesc d = b.descs[i];
        d.pair = partner[i] >= 0 ? 1 : 0;
        out.add(d, b.aux[b.descs[i].aux]);
        out.xinfo.push_back(b.xinfo[i]);
        if (partner[i] >= 0) {
            out.add(b.descs[(size_t)partner[i]], b.aux[b.descs[(size_t)partner[i]].aux]);
            out.xinfo.push_back(b.xinfo[(size_t)partner[i]]);
        }
    }
    b = std::move(out);
    return true;
}

bool spread_items(HostBatch& b, int ub, bool allow_pair) {
    if (b.descs.size() < 2 || b.descs.size() > (1u << (32 - kSpreadShift))) return false;
    for (const XInfo& x : b.xinfo)
        if (x.signal || x.wait) return false;
    for (const ReqDesc& d : b.descs)
        if (d.kind == K_LL || d.op == OP_SIGNAL) return false;
    if (allow_pair) pair_requests(b);
    const size_t n = b.descs.size();
    auto unpair = [&]() {
        for (ReqDesc& d : b.descs) d.pair = 0;
        return false;
    };
    std::vector<uint32_t> items(n);
    uint64_t total = 0;
    for (size_t r = 0; r < n; r++) {
        // the second member of a pair runs inside its partner's items
        items[r] = (r > 0 && b.descs[r - 1].pair) ? 0u : desc_items(b.descs[r], ub);
        if (items[r] > (1u << kSpreadShift)) return unpair();
        total += items[r];
    }
    // chunk c of request r at relative position (2c + 1) / (2 n_r); ties by r
    struct E { uint32_t r, c; };
    std::vector<E> e;
    e.reserve(total);
    for (size_t r = 0; r < n; r++)
        for (uint32_t c = 0; c < items[r]; c++) e.push_back(E{(uint32_t)r, c});
    std::stable_sort(e.begin(), e.end(), [&](const E& x, const E& y) {
        const uint64_t a = (2ull * x.c + 1) * items[y.r], c = (2ull * y.c + 1) * items[x.r];
        return a != c ? a < c : x.r < y.r;
    });
    b.gm.clear();
    b.order.resize(total);
    for (size_t i = 0; i < e.size(); i++) b.order[i] = (e[i].r << kSpreadShift) | e[i].c;
    return true;
}

size_t device_table_bytes(const HostBatch& b) {
    size_t n = b.descs.size();
    size_t off = sizeof(BatchHeader) + pad16((n + 1) * 4);
    if (!b.gm.empty()) off += pad16(n * 4);
    off += n * sizeof(ReqDesc) + b.aux.size() * sizeof(ReqDesc);
    if (!b.xinfo.empty()) off += n * sizeof(XInfo);
    off += b.order.size() * 4;
    return off;
}

// Variant 8: every descriptor moves 4-B vectors through a closed-form or
// uniform-list layout, at least one side is a list (the sparse configs[2]
// shape); items may then hold kUnrollNarrow vectors per thread.
static bool narrow_list_batch(const HostBatch& b) {
    const char* off = DDT_KNOB("DDT_NO_NARROW");  // experiments
    if (off && off[0] == '1') return false;
    bool list = false;
    for (const auto* v : {&b.descs, &b.aux})
        for (const ReqDesc& d : *v) {
            if (!d.nvec) continue;
            if (d.lw != 2 || d.ph) return false;
            if (d.kind == K_UNIFORM32 || d.kind == K_UNIFORM64) list = true;
            else if (d.kind != K_STRIDED && d.kind != K_CONTIG) return false;
        }
    return list && b.xinfo.empty();
}

// Variant 10 (segment per thread): every request moves 4-B vectors between a
// packed (contiguous) side and a uniform-list side whose segments hold the
// same vps <= 4 vectors (<= 16 B: the sparse configs[2] shape), no response
// slots.  Returns vps, or 0 if the batch does not qualify.
static int segment_batch_vps(const HostBatch& b) {
    const char* off = DDT_KNOB("DDT_NO_SEG");  // experiments
    if ((off && off[0] == '1') || !b.xinfo.empty()) return 0;
    uint32_t vps = 0;
    for (const ReqDesc& S : b.descs) {
        if (!S.nvec) continue;
        const ReqDesc& D = b.aux[S.aux];
        if (S.resp || S.lw != 2 || D.lw != 2 || S.ph || D.ph) return 0;
        const bool s_list = S.kind == K_UNIFORM32 || S.kind == K_UNIFORM64;
        const bool d_list = D.kind == K_UNIFORM32 || D.kind == K_UNIFORM64;
        const ReqDesc& L = s_list ? S : D;
        if (s_list == d_list || (s_list ? D.kind : S.kind) != K_CONTIG) return 0;
        if (L.vps.d == 0 || L.vps.d > 4 || (vps && L.vps.d != vps)) return 0;
        vps = L.vps.d;
    }
    return (int)vps;
}

int choose_ub(const HostBatch& b, int sm_count) {
    const char* env = DDT_KNOB("DDT_UB");
    if (env && (atoi(env) == 1 || atoi(env) == 2 || atoi(env) == 4 || atoi(env) == 8)) {
        const int u = atoi(env);
        return u == 8 && !narrow_list_batch(b) ? 4 : u;
    }
    const bool narrow = narrow_list_batch(b);
    for (int ub : {8, 4, 2}) {
        if (ub == 8 && !narrow) continue;
        uint64_t items = 0;
        for (const auto& d : b.descs) items += desc_items(d, ub);
        if (items >= 2ull * (uint64_t)sm_count) return ub;
    }
    return 1;
}

uint32_t write_device_table(void* dst, const HostBatch& b, int ub, uint64_t ticket, uint32_t claim) {
    size_t n = b.descs.size();
    auto* h = reinterpret_cast<BatchHeader*>(dst);
    std::memset(h, 0, sizeof(*h));
    h->ticket = ticket;
    h->claim = claim;
    auto* prefix = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(dst) + sizeof(BatchHeader));
    uint32_t items = fill_prefix(prefix, b, ub);
    if (!b.order.empty()) items = (uint32_t)b.order.size();  // spread: the item table (pairs share items)
    size_t off = sizeof(BatchHeader) + pad16((n + 1) * 4);
    if (!b.gm.empty()) {
        std::memcpy(reinterpret_cast<char*>(dst) + off, b.gm.data(), n * 4);
        off += pad16(n * 4);
    }
    h->ub = (uint32_t)ub;
    h->flags = batch_flags(b);
    h->nreq = (uint32_t)n;
    h->total_items = items;
    h->desc_offset = (uint32_t)off;
    std::memcpy(reinterpret_cast<char*>(dst) + off, b.descs.data(), n * sizeof(ReqDesc));
    off += n * sizeof(ReqDesc);
    h->aux_offset = (uint32_t)off;
    h->naux = (uint32_t)b.aux.size();
    if (!b.aux.empty()) std::memcpy(reinterpret_cast<char*>(dst) + off, b.aux.data(), b.aux.size() * sizeof(ReqDesc));
    off += b.aux.size() * sizeof(ReqDesc);
    if (!b.xinfo.empty()) {
        h->xinfo_offset = (uint32_t)off;
        std::memcpy(reinterpret_cast<char*>(dst) + off, b.xinfo.data(), n * sizeof(XInfo));
        off += n * sizeof(XInfo);
    }
    if (!b.order.empty()) {
        h->order_offset = (uint32_t)off;
        std::memcpy(reinterpret_cast<char*>(dst) + off, b.order.data(), b.order.size() * 4);
    }
    return items;
}

template <int CAP>
static void to_param(const HostBatch& b, Launchable& out) {
    // the kernel reads only the header and the first nreq entries of each
    // array: no per-flush zero-fill of the ~4-30 KB block (the first resize
    // zeroes it once)
    if (out.blob.size() != sizeof(ParamBatch<CAP>)) out.blob.assign(sizeof(ParamBatch<CAP>), 0);
    auto* p = reinterpret_cast<ParamBatch<CAP>*>(out.blob.data());
    std::memset(&p->h, 0, sizeof(p->h));
    p->h.nreq = (uint32_t)b.descs.size();
    p->h.ub = (uint32_t)out.ub;
    p->h.flags = batch_flags(b);
    p->h.total_items = fill_prefix(p->prefix, b, out.ub);
    p->h.ticket = out.ticket;
    p->h.claim = out.claim;
    std::copy(b.gm.begin(), b.gm.end(), p->gm);
    std::copy(b.descs.begin(), b.descs.end(), p->descs);
    std::copy(b.aux.begin(), b.aux.end(), p->aux);
    std::copy(b.xinfo.begin(), b.xinfo.end(), p->xinfo);
    out.total_items = p->h.total_items;
}

// The compact kernel variant applies when every source and destination
// descriptor is closed-form (strided or contiguous) with one vector width;
// batches holding a general list take variant 6 (shared-memory windows).
static int batch_variant(const HostBatch& b) {
    for (const auto* v : {&b.descs, &b.aux})
        for (const ReqDesc& d : *v)
            if (d.nvec && d.kind == K_GENERAL) return 6;
    for (const ReqDesc& d : b.descs)
        if (d.ph) return 7;  // phase_batch only phases strided-only batches
    if (narrow_list_batch(b)) return 8;
    int lw = -1;
    for (const ReqDesc& d : b.descs)
        if (d.nvec) {
            lw = d.lw;
            break;
        }
    if (lw < 0) return 0;
    for (const auto* v : {&b.descs, &b.aux})
        for (const ReqDesc& d : *v)
            if (d.nvec && ((d.kind != K_STRIDED && d.kind != K_CONTIG && d.kind != K_LL) || d.lw != lw)) return 0;
    return 1 + lw;
}

// Work distribution of a multi-wave plain batch (>= kTicketMinItemsPerSM
// items per SM, no exchange flags; exchange batches: see below).  Measured on
// one B200:
//   * spread halo plans (COMB) and sparse batches: one CTA per item (grid_mode 2)
//     -- COMB 128 -> 116 us, configs[2] 32 x 10^5 x 12 B 55 -> 52 us;
//   * <= kTicketMaxReqs large requests: dynamic tickets (grid_mode 1) --
//     16 x 64 MiB packs 5.5 -> 6.4 TB/s;
//   * many requests (1024 x 1 MiB): the static cyclic order stays best.
// Exchange batches (flags / LL windows) always claim items by ticket, in item
// order (fused_kernel.cu): one CTA per item (2) for one-wave plans, a
// resident-sized grid claiming chunks of items (1) for multi-wave ones
// (DDT_XGRID_MODE forces either).
static bool is_exchange_batch(const HostBatch& b) {
    for (const XInfo& x : b.xinfo)
        if (x.signal || x.wait) return true;
    for (const ReqDesc& d : b.descs)
        if (d.kind == K_LL || d.op == OP_SIGNAL) return true;
    return false;
}

static int grid_mode_for(const HostBatch& b, int ub, int sm_count) {
    const char* e = DDT_KNOB("DDT_GRID_MODE");  // experiments: force 0 / 1 / 2
    if (is_exchange_batch(b)) {
        const char* xe = DDT_KNOB("DDT_XGRID_MODE");
        uint64_t items = 0;
        for (const ReqDesc& d : b.descs) items += desc_items(d, d.xub ? d.xub : ub);
        int m = items > (uint64_t)kTicketMinItemsPerSM * (uint64_t)sm_count ? 1 : 2;
        if (xe && (xe[0] == '1' || xe[0] == '2')) m = xe[0] - '0';
        return m;
    }
    uint64_t items = 0;
    for (const ReqDesc& d : b.descs) items += desc_items(d, ub);
    if (items < (uint64_t)kTicketMinItemsPerSM * (uint64_t)sm_count) return 0;
    bool sparse = false;  // short-segment sides (sparse lists, halo x faces): DRAM-access bound
    for (const ReqDesc& d : b.descs) sparse |= d.l2_64 || b.aux[d.aux].l2_64;
    int m = (!b.order.empty() || sparse) ? 2 : (b.descs.size() <= (size_t)kTicketMaxReqs ? 1 : 0);
    if (e && e[0] >= '0' && e[0] <= '2') m = e[0] - '0';
    return (m == 1 && !b.ticket) ? 0 : m;
}

void make_launchable(const HostBatch& b, bool allow_param, Launchable& out, int sm_count, int force_ub) {
    size_t n = std::max(b.descs.size(), b.aux.size());
    out.variant = batch_variant(b);
    out.ub = force_ub > 0 ? force_ub : choose_ub(b, sm_count);
    if (const int vps = force_ub > 0 ? 0 : segment_batch_vps(b)) {
        // an item = kThreads x r0 whole segments (fewer if that leaves < 2 items per SM)
        out.variant = 10;
        out.ub = vps;
        const char* sr = DDT_KNOB("DDT_SEG_ROUNDS");  // experiments: segments per thread per item
        // 12-16-B segments: 2 per thread (more CTAs in flight; configs[2] sorted 52 -> 50 us,
        // shuffled 69 -> 58 us); 4-8-B segments: 4 (struct-on-indexed 4-B blocks 75 vs 89 us at 2)
        const int r0 = sr ? std::max(1, std::min(kSegUnroll, atoi(sr))) : (vps >= 3 ? 2 : kSegUnroll);
        for (int su : {r0, 1}) {
            uint64_t items = 0;
            for (const auto& d : b.descs) items += desc_items(d, vps * su);
            if (items >= 2ull * (uint64_t)sm_count) {
                out.ub = vps * su;
                break;
            }
        }
    }
    const char* v9 = DDT_KNOB("DDT_NO_V9");  // experiments
    bool multi = false;  // a request with its own item size > 1 needs the multi-slot kernel
    for (const ReqDesc& d : b.descs) multi |= d.xub > 1;
    if (out.variant == 7 && out.ub == 1 && !multi && !(v9 && v9[0] == '1')) out.variant = 9;
    if (is_exchange_batch(b) && (out.variant == 3 || out.variant == 4)) {  // exchange pairs: their own instance
        bool paired = false;
        for (const ReqDesc& d : b.descs) paired |= d.pair != 0;
        if (paired) out.variant += 8;
    }
    out.grid_mode = grid_mode_for(b, out.ub, sm_count);
    out.ticket = out.grid_mode == 1 ? b.ticket : 0;
    out.claim = 0;
    if (is_exchange_batch(b)) {
        // exchange kernels claim from the plan's tick (b.ticket = &XCtrl::tick):
        // one item per CTA (grid_mode 2, claim 0) or chunks of DDT_XCLAIM
        // (default kXClaim) consecutive items over a resident grid (grid_mode 1)
        out.ticket = b.ticket;
        const char* xc = DDT_KNOB("DDT_XCLAIM");
        const char* xg = DDT_KNOB("DDT_XONCE_G");  // items per CTA of one-wave exchange launches
        out.claim = out.grid_mode == 2 ? (kXOnce | (uint32_t)(xg ? std::max(1, std::min(64, atoi(xg))) : 1))
                                       : (uint32_t)(xc ? std::max(1, atoi(xc)) : kXClaim);
    }
    const char* force = DDT_KNOB("DDT_FORCE_TABLE");  // experiments: always use the device-table form
    if (force && force[0] == '1') allow_param = false;
    const char* large = DDT_KNOB("DDT_FORCE_LARGE_PARAM");  // experiments: skip the small parameter form
    const bool skip_small = large && large[0] == '1';
    if (allow_param && n <= (size_t)kParamSmall && !skip_small) {
        out.form = 1;
        to_param<kParamSmall>(b, out);
    } else if (allow_param && n <= (size_t)kParamLarge) {
        out.form = 2;
        to_param<kParamLarge>(b, out);
    } else {
        out.form = 3;
        out.blob.clear();
        std::vector<uint32_t> prefix(b.descs.size() + 1);
        out.total_items = fill_prefix(prefix.data(), b, out.ub);
        if (!b.order.empty()) out.total_items = (uint32_t)b.order.size();
    }
}

int launch_fused(const Launchable& l, void* stream, int grid_cap) {
    const void* src = l.form == 3 ? l.dev : (const void*)l.blob.data();
    if (l.grid_mode == 2 && grid_cap <= 0) grid_cap = -1;  // one CTA per item
    return launch_fused_form(l.form, l.variant, src, l.total_items, stream, grid_cap);
}

int launch_exchange(const Launchable& l, const XArgs& xa, void* stream, int grid_cap) {
    const void* src = l.form == 3 ? l.dev : (const void*)l.blob.data();
    if (l.grid_mode == 2 && grid_cap <= 0) {  // one claim of G items per CTA: grid = ceil(items / G)
        const uint32_t G = std::max(1u, l.claim & ~kXOnce);
        grid_cap = -(int)((l.total_items + G - 1) / G);
    }
    return launch_exchange_form(l.form, l.variant, src, l.total_items, xa, stream, grid_cap);
}

}  // namespace ddt
