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

static uint32_t fill_prefix(uint32_t* prefix, const std::vector<ReqDesc>& d, int ub) {
    uint64_t acc = 0;
    for (size_t i = 0; i < d.size(); i++) {
        prefix[i] = (uint32_t)acc;
        acc += desc_items(d[i], ub);
    }
    prefix[d.size()] = (uint32_t)acc;
    return (uint32_t)acc;
}

static size_t pad16(size_t v) { return (v + 15) & ~(size_t)15; }

// Item order (experiments: DDT_ITEM_ORDER=blocked); cyclic is the default.
static uint32_t item_order_blocked() {
    const char* e = getenv("DDT_ITEM_ORDER");
    return (e && e[0] == 'b') ? 1u : 0u;
}

size_t device_table_bytes(const HostBatch& b) {
    size_t n = b.descs.size();
    size_t off = sizeof(BatchHeader) + pad16((n + 1) * 4);
    off += n * sizeof(ReqDesc) + b.aux.size() * sizeof(ReqDesc);
    if (!b.xinfo.empty()) off += n * sizeof(XInfo);
    return off;
}

int choose_ub(const HostBatch& b, int sm_count) {
    const char* env = getenv("DDT_UB");
    if (env && (atoi(env) == 1 || atoi(env) == 2 || atoi(env) == 4)) return atoi(env);
    for (int ub : {4, 2}) {
        uint64_t items = 0;
        for (const auto& d : b.descs) items += desc_items(d, ub);
        if (items >= 2ull * (uint64_t)sm_count) return ub;
    }
    return 1;
}

uint32_t write_device_table(void* dst, const HostBatch& b, int ub) {
    size_t n = b.descs.size();
    auto* h = reinterpret_cast<BatchHeader*>(dst);
    std::memset(h, 0, sizeof(*h));
    auto* prefix = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(dst) + sizeof(BatchHeader));
    uint32_t items = fill_prefix(prefix, b.descs, ub);
    size_t off = sizeof(BatchHeader) + pad16((n + 1) * 4);
    h->ub = (uint32_t)ub;
    h->blocked = item_order_blocked();
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
    }
    return items;
}

template <int CAP>
static void to_param(const HostBatch& b, Launchable& out) {
    out.blob.assign(sizeof(ParamBatch<CAP>), 0);
    auto* p = reinterpret_cast<ParamBatch<CAP>*>(out.blob.data());
    p->h.nreq = (uint32_t)b.descs.size();
    p->h.ub = (uint32_t)out.ub;
    p->h.blocked = item_order_blocked();
    p->h.total_items = fill_prefix(p->prefix, b.descs, out.ub);
    std::copy(b.descs.begin(), b.descs.end(), p->descs);
    std::copy(b.aux.begin(), b.aux.end(), p->aux);
    std::copy(b.xinfo.begin(), b.xinfo.end(), p->xinfo);
    out.total_items = p->h.total_items;
}

// The compact kernel variant applies when every source and destination
// descriptor is closed-form (strided or contiguous) with one vector width.
static int batch_variant(const HostBatch& b) {
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

void make_launchable(const HostBatch& b, bool allow_param, Launchable& out, int sm_count, int force_ub) {
    size_t n = std::max(b.descs.size(), b.aux.size());
    out.variant = batch_variant(b);
    out.ub = force_ub > 0 ? force_ub : choose_ub(b, sm_count);
    out.blob.clear();
    const char* force = getenv("DDT_FORCE_TABLE");  // experiments: always use the device-table form
    if (force && force[0] == '1') allow_param = false;
    const char* large = getenv("DDT_FORCE_LARGE_PARAM");  // experiments: skip the small parameter form
    const bool skip_small = large && large[0] == '1';
    if (allow_param && n <= (size_t)kParamSmall && !skip_small) {
        out.form = 1;
        to_param<kParamSmall>(b, out);
    } else if (allow_param && n <= (size_t)kParamLarge) {
        out.form = 2;
        to_param<kParamLarge>(b, out);
    } else {
        out.form = 3;
        std::vector<uint32_t> prefix(b.descs.size() + 1);
        out.total_items = fill_prefix(prefix.data(), b.descs, out.ub);
    }
}

int launch_fused(const Launchable& l, void* stream, int grid_cap) {
    const void* src = l.form == 3 ? l.dev : (const void*)l.blob.data();
    return launch_fused_form(l.form, l.variant, src, l.total_items, stream, grid_cap);
}

int launch_exchange(const Launchable& l, const XArgs& xa, void* stream, int grid_cap) {
    const void* src = l.form == 3 ? l.dev : (const void*)l.blob.data();
    return launch_exchange_form(l.form, l.variant, src, l.total_items, xa, stream, grid_cap);
}

}  // namespace ddt
