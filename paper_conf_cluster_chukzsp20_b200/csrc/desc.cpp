// desc.cpp -- one request -> one device descriptor (the per-request part of
// the paper's request object, §IV-A.1: operation, origin / target
// buffer, cached data layout entry), built once at enqueue in O(1) from the
// committed layout cache.  All address arithmetic is signed 64-bit; the
// vector width is the largest power of two (<= 16 B) dividing every offset,
// length and pointer involved, so every device access is naturally aligned.
#include <algorithm>
#include <cstring>

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
                        int64_t count, ReqDesc* d, int max_lw) {
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
    if (lw > max_lw) lw = max_lw;
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


static int desc_lw_uncapped(ddt_type_s* t, const void* nc, const void* pk, int64_t count) {
    int w = t->layout.align;
    w = std::min(w, lowbit16((uint64_t)(uintptr_t)nc));
    if (pk) w = std::min(w, lowbit16((uint64_t)(uintptr_t)pk));
    if (count > 1) w = std::min(w, lowbit16(uabs64(type_extent(t))));
    int lw = 0;
    while ((1 << lw) < w) lw++;
    return lw;
}

// DirectIPC: gather through the source layout and scatter
// through the destination layout in one pass (no packed intermediate).  Both
// descriptors share one vector width and vector count; `d` carries the items.
ddt_status_t build_direct(ddt_type_s* ts, const DeviceLayout* dls, const void* src, int64_t scount, ddt_type_s* td,
                          const DeviceLayout* dld, void* dst, int64_t dcount, ReqDesc* d, ReqDesc* a) {
    if (scount * ts->size != dcount * td->size) return DDT_ERR_SIZE_MISMATCH;
    int lw = std::min(desc_lw_uncapped(ts, src, nullptr, scount), desc_lw_uncapped(td, dst, nullptr, dcount));
    ddt_status_t s = build_desc(ts, dls, OP_DIRECT, src, nullptr, scount, d, lw);
    if (s != DDT_OK) return s;
    s = build_desc(td, dld, OP_DIRECT, dst, nullptr, dcount, a, lw);
    if (s != DDT_OK) return s;
    if (d->nvec != a->nvec || d->lw != a->lw) return DDT_ERR_STATE;
    return DDT_OK;
}

}  // namespace ddt
