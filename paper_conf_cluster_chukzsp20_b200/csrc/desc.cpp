// desc.cpp -- one request -> a (source, destination) pair of device layout
// descriptors (the per-request part of the paper's request object, §IV-A.1
// operation, origin / target buffer, cached data layout entry),
// built once at enqueue in O(1) from the committed layout cache.
//
// Every operation is "load vector v through the source layout, store it
// through the destination layout":
//   pack   = (type layout over the origin buffer) -> (contiguous packed buffer)
//   unpack = (contiguous packed buffer)           -> (type layout over the target)
//   direct = (source type layout)                 -> (destination type layout)
//            -- the paper's DirectIPC op, no packed intermediate.
// All address arithmetic is signed 64-bit; the vector width w is the largest
// power of two (<= 16 B) dividing every segment offset and length, both
// pointers and (count > 1) the extent, so every device access is naturally
// aligned and the two sides of a pair always share one width.
#include <algorithm>
#include <cstdlib>
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

static int log2i(int w) {
    int lw = 0;
    while ((1 << lw) < w) lw++;
    return lw;
}

// Largest legal log2 vector width of one side (type layout over pointer p).
int side_lw(ddt_type_s* t, const void* p, int64_t count) {
    int w = std::min(t->layout.align, lowbit16((uint64_t)(uintptr_t)p));
    if (count > 1) w = std::min(w, lowbit16(uabs64(type_extent(t))));
    return log2i(w);
}

// experiments: DDT_NO_L2HINT=1 disables the sparse-side prefetch-size hint
static bool l2_hint_on() {
    static const bool on = [] {
        const char* e = DDT_KNOB("DDT_NO_L2HINT");
        return !(e && e[0] == '1');
    }();
    return on;
}

// Fill the layout fields of `d` for `count` instances of t at `base_ptr`.
static ddt_status_t layout_desc(ddt_type_s* t, const DeviceLayout* dl, const void* base_ptr, int64_t count, int lw,
                                ReqDesc* d) {
    const Layout& L = t->layout;
    int64_t bytes = count * t->size;
    int64_t ext = type_extent(t);
    uint64_t nvec = (uint64_t)bytes >> lw;
    if (nvec >= (1ull << 32)) {
        set_error("request too large for one descriptor (>= 2^32 vectors)");
        return DDT_ERR_UNSUPPORTED;
    }
    d->ptr = (uint64_t)(uintptr_t)base_ptr;
    d->nvec = (uint32_t)nvec;
    d->lw = (uint8_t)lw;
    d->extent = ext;
    if (L.kind == DDT_LAYOUT_STRIDED) {
        // dims = [(count, extent)] ++ layout dims, normalised without heap
        // allocation (the same rules as normalize(): drop unit dims, fold a
        // contiguous innermost dim into the segment, merge chained dims)
        Dim dims[kMaxDims + 2];
        int D = 0;
        int64_t seg = L.form.seg_len;
        if (count != 1) dims[D++] = Dim{count, ext};
        for (const Dim& x : L.form.dims)
            if (x.n != 1) dims[D++] = x;
        bool changed = true;
        while (changed) {
            changed = false;
            if (D > 0 && dims[D - 1].stride == seg) {
                seg *= dims[D - 1].n;
                D--;
                changed = true;
                continue;
            }
            for (int k = 0; k + 1 < D; k++) {
                if (dims[k].stride == dims[k + 1].n * dims[k + 1].stride) {
                    dims[k + 1].n *= dims[k].n;
                    for (int j = k; j + 1 < D; j++) dims[j] = dims[j + 1];
                    D--;
                    changed = true;
                    break;
                }
            }
        }
        d->kind = K_STRIDED;
        d->base = L.form.base;
        d->vps = make_div((uint32_t)(seg >> lw));
        d->l2_64 = (D > 0 && seg < kSparseSeg && l2_hint_on()) ? 1 : 0;
        if (D == 0) {
            if (d->base == 0) d->kind = K_CONTIG;  // one contiguous run at the pointer itself
            d->ndim = 0;
            d->extent = 0;
        } else {
            if (D - 1 > kMaxDims) {
                set_error("strided layout with too many dims after count folding");
                return DDT_ERR_UNSUPPORTED;
            }
            d->ndim = (uint8_t)(D - 1);
            // innermost first; the outermost dim is the final quotient (no division)
            for (int k = 0; k < D - 1; k++) {
                const Dim& x = dims[D - 1 - k];
                d->radix[k] = make_div((uint32_t)x.n);
                d->stride[k] = x.stride;
            }
            d->extent = dims[0].stride;
        }
    } else if (L.kind == DDT_LAYOUT_UNIFORM_LIST) {
        d->kind = L.off32 ? K_UNIFORM32 : K_UNIFORM64;
        d->l2_64 = (L.seg_len < kSparseSeg && l2_hint_on()) ? 1 : 0;
        d->vps = make_div((uint32_t)(L.seg_len >> lw));
        d->nseg = make_div((uint32_t)L.nseg);
        d->list = (uint64_t)(uintptr_t)dl->offsets;
    } else if (L.kind == DDT_LAYOUT_GENERAL_LIST) {
        d->kind = K_GENERAL;
        d->l2_64 = (L.nseg > 0 && t->size < kSparseSeg * L.nseg && l2_hint_on()) ? 1 : 0;  // mean segment shorter than kSparseSeg
        d->vps = make_div((uint32_t)(t->size >> lw));  // vectors per instance
        d->list = (uint64_t)(uintptr_t)dl->offsets;
        d->skip = (uint64_t)(uintptr_t)dl->skip;
        d->prefix = (uint64_t)(uintptr_t)dl->prefix;
        d->list_n = (uint32_t)L.nseg;
    } else {
        return DDT_ERR_STATE;
    }
    return DDT_OK;
}

static void contig_desc(const void* p, uint32_t nvec, int lw, ReqDesc* d) {
    std::memset(d, 0, sizeof(*d));
    d->ptr = (uint64_t)(uintptr_t)p;
    d->nvec = nvec;
    d->lw = (uint8_t)lw;
    d->kind = K_CONTIG;
}

ddt_status_t build_request(int op, ddt_type_s* t, const DeviceLayout* dl, const void* src, const void* dst,
                           int64_t count, ReqDesc* s, ReqDesc* d) {
    const void* nc = op == OP_PACK ? src : dst;  // the typed side
    const void* pk = op == OP_PACK ? dst : src;  // the packed side
    int lw = std::min(side_lw(t, nc, count), log2i(lowbit16((uint64_t)(uintptr_t)pk)));
    ReqDesc* lay = op == OP_PACK ? s : d;  // built in place: no temporaries
    ReqDesc* con = op == OP_PACK ? d : s;
    std::memset(lay, 0, sizeof(*lay));
    ddt_status_t st = layout_desc(t, dl, nc, count, lw, lay);
    if (st != DDT_OK) return st;
    contig_desc(pk, lay->nvec, lw, con);
    s->op = (uint8_t)op;
    d->op = (uint8_t)op;
    return DDT_OK;
}

ddt_status_t build_direct(ddt_type_s* ts, const DeviceLayout* dls, const void* src, int64_t scount, ddt_type_s* td,
                          const DeviceLayout* dld, void* dst, int64_t dcount, ReqDesc* s, ReqDesc* d) {
    if (scount * ts->size != dcount * td->size) return DDT_ERR_SIZE_MISMATCH;
    std::memset(s, 0, sizeof(*s));
    std::memset(d, 0, sizeof(*d));
    int lw = std::min(side_lw(ts, src, scount), side_lw(td, dst, dcount));
    ddt_status_t st = layout_desc(ts, dls, src, scount, lw, s);
    if (st == DDT_OK) st = layout_desc(td, dld, dst, dcount, lw, d);
    if (st != DDT_OK) return st;
    if (s->nvec != d->nvec) return DDT_ERR_STATE;
    s->op = d->op = OP_DIRECT;
    return DDT_OK;
}

// A typed descriptor at its own largest legal width (pack-free remote
// transfers: the receiver publishes its destination side, the sender
// rescales both sides to their common width).
ddt_status_t build_typed(ddt_type_s* t, const DeviceLayout* dl, const void* p, int64_t count, ReqDesc* d) {
    std::memset(d, 0, sizeof(*d));
    return layout_desc(t, dl, p, count, side_lw(t, p, count), d);
}

// LL exchange request: the typed side at 8-B vectors, the window side in LL
// format (16 B per vector).  Needs a typed side whose width allows 8 B.
ddt_status_t build_ll(int op, ddt_type_s* t, const DeviceLayout* dl, const void* typed, const void* window,
                      int64_t count, ReqDesc* s, ReqDesc* d) {
    ReqDesc ty, ll;
    ddt_status_t st = build_typed(t, dl, typed, count, &ty);
    if (st != DDT_OK) return st;
    if (ty.lw < 3) return DDT_ERR_UNSUPPORTED;
    if (ty.lw > 3 && (st = rescale_desc(&ty, 3)) != DDT_OK) return st;
    std::memset(&ll, 0, sizeof(ll));
    ll.ptr = (uint64_t)(uintptr_t)window;
    ll.nvec = ty.nvec;
    ll.lw = 3;
    ll.kind = K_LL;
    *s = op == OP_PACK ? ty : ll;
    *d = op == OP_PACK ? ll : ty;
    s->op = d->op = (uint8_t)op;
    return DDT_OK;
}

// Re-express a closed-form descriptor at a smaller vector width.
ddt_status_t rescale_desc(ReqDesc* d, int lw) {
    if (lw > d->lw) return DDT_ERR_ARG;
    if (d->kind != K_STRIDED && d->kind != K_CONTIG) return DDT_ERR_UNSUPPORTED;
    const int sh = d->lw - lw;
    uint64_t nvec = (uint64_t)d->nvec << sh;
    uint64_t vps = (uint64_t)d->vps.d << sh;
    if (nvec >= (1ull << 32) || vps >= (1ull << 32)) return DDT_ERR_UNSUPPORTED;
    d->nvec = (uint32_t)nvec;
    if (d->kind == K_STRIDED) d->vps = make_div((uint32_t)vps);
    d->lw = (uint8_t)lw;
    return DDT_OK;
}

}  // namespace ddt
