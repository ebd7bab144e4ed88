// types.cpp -- MPI-style datatype construction, closed-form size / bounds, and
// the flattener that fills the layout cache at commit.
//
// Paper: datatypes are created and committed once (Alg 1 lines 1-2 P:102-103,
// Alg 3 lines 1-2 P:169-170); the runtime keeps a "cached data layout entry"
// per datatype (§IV-A.1, §IV-B.1, Table I "Layout Cache" P:46).
// Semantics are MPI-3.1 §4.1 (ref [29]).  The layout-cache format is not
// given in the paper (it points to [24]); ours is DESIGN.md reading R7.
//
// Closed forms used here (the oracle derives the same quantities by
// enumeration, so tests pin one against the other):
//   vector/hvector (S = stride bytes, E = ext(old), c,b > 0):
//     lb = min(0,(c-1)S) + lb(old),  ub = max(0,(c-1)S) + (b-1)E + ub(old)
//   indexed/hindexed over blocks with B_i > 0 (d_i in bytes):
//     lb = min_i d_i + lb(old),      ub = max_i (d_i + (B_i-1)E) + ub(old)
//   subarray: lb = 0, ub = prod(sizes) * E (resized, MPI-3.1 §4.1.3)
//   size: c*b*size(old), sum(B)*size(old), prod(subsizes)*size(old)
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <numeric>

#include <cuda_runtime.h>

#include "ddt_internal.h"

namespace ddt {

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;
void set_error(const std::string& msg) { g_err = msg; }
const char* last_error() { return g_err.c_str(); }
ddt_status_t cuda_fail(const char* what, int err) {
    set_error(std::string(what) + ": " + cudaGetErrorString((cudaError_t)err));
    return DDT_ERR_CUDA;
}

// ------------------------------------------------------------------ forms
int64_t Form::num_segments() const {
    int64_t n = 1;
    for (auto& d : dims) n *= d.n;
    return n;
}

bool normalize(Form& f) {
    if (f.seg_len <= 0) return false;
    for (auto& d : f.dims)
        if (d.n <= 0) return false;
    bool changed = true;
    while (changed) {
        changed = false;
        // unit dims contribute nothing
        auto it = std::remove_if(f.dims.begin(), f.dims.end(), [](const Dim& d) { return d.n == 1; });
        if (it != f.dims.end()) { f.dims.erase(it, f.dims.end()); changed = true; }
        // innermost dim contiguous with the segment -> longer segment
        if (!f.dims.empty() && f.dims.back().stride == f.seg_len) {
            f.seg_len *= f.dims.back().n;
            f.dims.pop_back();
            changed = true;
            continue;
        }
        // outer dim stride == inner extent -> one dim (row-major order preserved)
        for (size_t d = 0; d + 1 < f.dims.size(); d++) {
            if (f.dims[d].stride == f.dims[d + 1].n * f.dims[d + 1].stride) {
                f.dims[d + 1].n *= f.dims[d].n;
                f.dims.erase(f.dims.begin() + (long)d);
                changed = true;
                break;
            }
        }
    }
    return true;
}

static int64_t lowbit_align(uint64_t v) {
    // largest power of two <= 16 dividing v (v == 0 -> 16)
    if (v == 0) return 16;
    int64_t a = (int64_t)(v & (~v + 1));
    return a > 16 ? 16 : a;
}

static uint64_t uabs(int64_t v) { return v < 0 ? (uint64_t)(-(v + 1)) + 1 : (uint64_t)v; }

// ---------------------------------------------------------------- refcount
void type_retain(ddt_type_s* t) {
    if (t && !t->predefined) t->refs.fetch_add(1);
}

static void free_device_layouts(ddt_type_s* t) {
    int cur = -1;
    if (t->dev.empty()) return;
    cudaGetDevice(&cur);
    for (auto& kv : t->dev) {
        cudaSetDevice(kv.first);
        cudaFree(kv.second.offsets);
        cudaFree(kv.second.lens);
        cudaFree(kv.second.prefix);
        cudaFree(kv.second.skip);
    }
    if (cur >= 0) cudaSetDevice(cur);
}

void type_release(ddt_type_s* t) {
    if (!t || t->predefined) return;
    if (t->refs.fetch_sub(1) == 1) {
        ddt_type_s* old = t->old;
        std::vector<ddt_type_s*> kids;
        kids.swap(t->types);
        free_device_layouts(t);
        delete t;
        type_release(old);
        for (ddt_type_s* k : kids) type_release(k);
    }
}

// ----------------------------------------------------------- basic types
static ddt_type_s* g_basic[5];
static std::once_flag g_basic_once;

static void init_basic() {
    static const int64_t sz[5] = {1, 4, 8, 4, 8};
    for (int i = 0; i < 5; i++) {
        auto* t = new ddt_type_s();
        t->kind = T_BASIC;
        t->base = i;
        t->predefined = true;
        t->elem = sz[i];
        t->nonempty = true;
        t->size = sz[i];
        t->lb = 0;
        t->ub = sz[i];
        t->true_lb = 0;
        t->true_ub = sz[i];
        t->align = sz[i];
        t->has_form = true;
        t->form.base = 0;
        t->form.seg_len = sz[i];
        g_basic[i] = t;
    }
}

// Place `old` at the copy displacements described by (pbase, pdims) and
// derive size / bounds / form.  ncopies > 0 unless the constructor is empty.
static void derive_from_copies(ddt_type_s* t, int64_t ncopies, int64_t min_disp, int64_t max_disp,
                               int64_t pbase, const std::vector<Dim>* pdims) {
    ddt_type_s* o = t->old;
    t->size = ncopies * o->size;
    t->nonempty = ncopies > 0 && o->nonempty;
    t->align = o->align;
    t->sticky = o->sticky;
    if (!t->nonempty) {
        t->lb = t->ub = t->true_lb = t->true_ub = 0;
        t->has_form = true;
        t->form = Form();
        return;
    }
    t->lb = min_disp + o->lb;
    t->ub = max_disp + o->ub;
    t->true_lb = min_disp + o->true_lb;
    t->true_ub = max_disp + o->true_ub;
    if (pdims && o->has_form) {
        Form f;
        f.base = pbase + o->form.base;
        f.seg_len = o->form.seg_len;
        f.dims = *pdims;
        f.dims.insert(f.dims.end(), o->form.dims.begin(), o->form.dims.end());
        t->has_form = normalize(f);
        t->form = f;
    } else {
        t->has_form = false;
    }
}

static ddt_type_s* new_derived(int kind, ddt_type_s* old) {
    auto* t = new ddt_type_s();
    t->kind = kind;
    t->old = old;
    type_retain(old);
    return t;
}

static void derive_vector_like(ddt_type_s* t, int64_t c, int64_t b, int64_t S) {
    int64_t E = type_extent(t->old);
    int64_t ncopies = c * b;
    int64_t mn = std::min<int64_t>(0, (c - 1) * S);
    int64_t mx = std::max<int64_t>(0, (c - 1) * S) + (b - 1) * E;
    std::vector<Dim> dims = {{c, S}, {b, E}};
    derive_from_copies(t, ncopies, mn, mx, 0, &dims);
}

static void derive_indexed_like(ddt_type_s* t, bool bytes) {
    int64_t E = type_extent(t->old);
    int64_t ncopies = 0;
    bool any = false;
    int64_t mn = 0, mx = 0;
    // regular (uniform block length, arithmetic displacements) -> strided form
    std::vector<std::pair<int64_t, int64_t>> nz;  // (disp bytes, blocklen)
    for (size_t i = 0; i < t->blocklens.size(); i++) {
        int64_t B = t->blocklens[i];
        if (B <= 0) continue;
        int64_t d = bytes ? t->displs[i] : t->displs[i] * E;
        ncopies += B;
        int64_t lo = d, hi = d + (B - 1) * E;
        if (!any || lo < mn) mn = lo;
        if (!any || hi > mx) mx = hi;
        any = true;
        nz.push_back({d, B});
    }
    bool regular = !nz.empty();
    int64_t delta = nz.size() > 1 ? nz[1].first - nz[0].first : 0;
    for (size_t i = 0; regular && i < nz.size(); i++) {
        if (nz[i].second != nz[0].second) regular = false;
        if (i > 0 && nz[i].first - nz[i - 1].first != delta) regular = false;
    }
    if (regular) {
        std::vector<Dim> dims = {{(int64_t)nz.size(), delta}, {nz[0].second, E}};
        derive_from_copies(t, ncopies, mn, mx, nz[0].first, &dims);
    } else {
        derive_from_copies(t, ncopies, mn, mx, 0, nullptr);
    }
}

static void derive_subarray(ddt_type_s* t) {
    int64_t E = type_extent(t->old);
    int nd = t->ndims;
    std::vector<int64_t> mult(nd, 1);
    for (int k = 0; k < nd; k++) {
        int64_t m = 1;
        if (t->order == DDT_ORDER_C) {
            for (int q = k + 1; q < nd; q++) m *= t->sizes[q];
        } else {
            for (int q = 0; q < k; q++) m *= t->sizes[q];
        }
        mult[k] = m * E;
    }
    int64_t ncopies = 1, mn = 0, mx = 0, full = 1;
    for (int k = 0; k < nd; k++) {
        ncopies *= t->subsizes[k];
        mn += t->starts[k] * mult[k];
        mx += (t->starts[k] + t->subsizes[k] - 1) * mult[k];
        full *= t->sizes[k];
    }
    std::vector<Dim> dims;
    if (t->order == DDT_ORDER_C) {
        for (int k = 0; k < nd; k++) dims.push_back({t->subsizes[k], mult[k]});
    } else {
        for (int k = nd - 1; k >= 0; k--) dims.push_back({t->subsizes[k], mult[k]});
    }
    derive_from_copies(t, ncopies, mn, mx, mn, &dims);
    t->sticky = true;  // defined with explicit bounds (MPI-3.1 §4.1.3)
    // resized: lb 0, extent prod(sizes) * E (true bounds are the entries')
    if (t->nonempty) {
        t->lb = 0;
        t->ub = full * E;
    }
}

// struct: block i = blocklens[i] copies of types[i] at displs[i] + j*ext(types[i])
// (byte displacements, MPI-3.1 §4.1.2).  Alignment epsilon (reading R2): ub is
// rounded up so that the extent is a multiple of the largest basic alignment in
// the typemap, unless a child carries explicit bounds (resized / subarray).
static void derive_struct(ddt_type_s* t) {
    bool any = false;
    int64_t lb = 0, ub = 0, tlb = 0, tub = 0;
    t->size = 0;
    t->align = 1;
    t->sticky = false;
    for (size_t i = 0; i < t->blocklens.size(); i++) {
        const ddt_type_s* o = t->types[i];
        int64_t B = t->blocklens[i];
        t->size += B * o->size;
        t->sticky |= o->sticky;
        if (B <= 0 || !o->nonempty) continue;
        t->align = std::max(t->align, o->align);
        int64_t E = type_extent(o), d = t->displs[i];
        int64_t blo = d + o->lb, bhi = d + (B - 1) * E + o->ub;
        int64_t tlo = d + o->true_lb, thi = d + (B - 1) * E + o->true_ub;
        if (!any || blo < lb) lb = blo;
        if (!any || bhi > ub) ub = bhi;
        if (!any || tlo < tlb) tlb = tlo;
        if (!any || thi > tub) tub = thi;
        any = true;
    }
    t->nonempty = any;
    if (!any) {
        t->lb = t->ub = t->true_lb = t->true_ub = 0;
        t->has_form = true;
        t->form = Form();
        return;
    }
    t->lb = lb;
    t->ub = ub;
    if (!t->sticky) {
        const int64_t ext = ub - lb;
        t->ub += (t->align - ext % t->align) % t->align;  // epsilon
    }
    t->true_lb = tlb;
    t->true_ub = tub;
    // one non-empty block of a closed-form oldtype is itself closed-form
    int nz = -1, cnt = 0;
    for (size_t i = 0; i < t->blocklens.size(); i++)
        if (t->blocklens[i] > 0 && t->types[i]->nonempty) {
            nz = (int)i;
            cnt++;
        }
    t->has_form = false;
    if (cnt == 1 && t->types[(size_t)nz]->has_form) {
        const ddt_type_s* o = t->types[(size_t)nz];
        Form f;
        f.base = t->displs[(size_t)nz] + o->form.base;
        f.seg_len = o->form.seg_len;
        f.dims.push_back({t->blocklens[(size_t)nz], type_extent(o)});
        f.dims.insert(f.dims.end(), o->form.dims.begin(), o->form.dims.end());
        t->has_form = normalize(f);
        t->form = f;
    }
}

}  // namespace ddt

using namespace ddt;

// ================================================================== C ABI
extern "C" {

ddt_status_t ddt_type_basic(int base, ddt_type_t* out) {
    if (!out || base < 0 || base > 4) return DDT_ERR_ARG;
    std::call_once(g_basic_once, init_basic);
    *out = g_basic[base];
    return DDT_OK;
}

ddt_status_t ddt_create_contiguous(int64_t count, ddt_type_t old, ddt_type_t* out) {
    if (!out || !old || count < 0) return DDT_ERR_ARG;
    auto* t = new_derived(T_CONTIG, old);
    t->count = count;
    derive_vector_like(t, count > 0 ? 1 : 0, count, 0);
    *out = t;
    return DDT_OK;
}

ddt_status_t ddt_create_vector(int64_t count, int64_t blocklen, int64_t stride, ddt_type_t old, ddt_type_t* out) {
    if (!out || !old || count < 0 || blocklen < 0) return DDT_ERR_ARG;
    auto* t = new_derived(T_VECTOR, old);
    t->count = count;
    t->blocklen = blocklen;
    t->stride = stride;
    derive_vector_like(t, count, blocklen, stride * type_extent(old));
    *out = t;
    return DDT_OK;
}

ddt_status_t ddt_create_hvector(int64_t count, int64_t blocklen, int64_t stride_bytes, ddt_type_t old,
                                ddt_type_t* out) {
    if (!out || !old || count < 0 || blocklen < 0) return DDT_ERR_ARG;
    auto* t = new_derived(T_HVECTOR, old);
    t->count = count;
    t->blocklen = blocklen;
    t->stride = stride_bytes;
    derive_vector_like(t, count, blocklen, stride_bytes);
    *out = t;
    return DDT_OK;
}

static ddt_status_t create_indexed(int kind, int64_t count, const int64_t* bl, const int64_t* d, ddt_type_t old,
                                   ddt_type_t* out) {
    if (!out || !old || count < 0 || (count > 0 && (!bl || !d))) return DDT_ERR_ARG;
    for (int64_t i = 0; i < count; i++)
        if (bl[i] < 0) return DDT_ERR_ARG;
    auto* t = new_derived(kind, old);
    t->blocklens.assign(bl, bl + count);
    t->displs.assign(d, d + count);
    derive_indexed_like(t, kind == T_HINDEXED);
    *out = t;
    return DDT_OK;
}

ddt_status_t ddt_create_indexed(int64_t count, const int64_t* blocklens, const int64_t* displs, ddt_type_t old,
                                ddt_type_t* out) {
    return create_indexed(T_INDEXED, count, blocklens, displs, old, out);
}

ddt_status_t ddt_create_hindexed(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes,
                                 ddt_type_t old, ddt_type_t* out) {
    return create_indexed(T_HINDEXED, count, blocklens, displs_bytes, old, out);
}

ddt_status_t ddt_create_subarray(int ndims, const int64_t* sizes, const int64_t* subsizes, const int64_t* starts,
                                 int order, ddt_type_t old, ddt_type_t* out) {
    if (!out || !old || ndims < 1 || ndims > 16 || !sizes || !subsizes || !starts) return DDT_ERR_ARG;
    if (order != DDT_ORDER_C && order != DDT_ORDER_FORTRAN) return DDT_ERR_ARG;
    for (int k = 0; k < ndims; k++) {
        if (sizes[k] < 1 || subsizes[k] < 1 || subsizes[k] > sizes[k] || starts[k] < 0 ||
            starts[k] > sizes[k] - subsizes[k])
            return DDT_ERR_ARG;
    }
    auto* t = new_derived(T_SUBARRAY, old);
    t->ndims = ndims;
    t->order = order;
    t->sizes.assign(sizes, sizes + ndims);
    t->subsizes.assign(subsizes, subsizes + ndims);
    t->starts.assign(starts, starts + ndims);
    derive_subarray(t);
    *out = t;
    return DDT_OK;
}

ddt_status_t ddt_create_indexed_block(int64_t count, int64_t blocklen, const int64_t* displs, ddt_type_t old,
                                      ddt_type_t* out) {
    if (count < 0 || blocklen < 0) return DDT_ERR_ARG;
    std::vector<int64_t> bl((size_t)count, blocklen);
    return create_indexed(T_INDEXED, count, bl.data(), displs, old, out);
}

ddt_status_t ddt_create_hindexed_block(int64_t count, int64_t blocklen, const int64_t* displs_bytes, ddt_type_t old,
                                       ddt_type_t* out) {
    if (count < 0 || blocklen < 0) return DDT_ERR_ARG;
    std::vector<int64_t> bl((size_t)count, blocklen);
    return create_indexed(T_HINDEXED, count, bl.data(), displs_bytes, old, out);
}

ddt_status_t ddt_create_struct(int64_t count, const int64_t* blocklens, const int64_t* displs_bytes,
                               const ddt_type_t* types, ddt_type_t* out) {
    if (!out || count < 0 || (count > 0 && (!blocklens || !displs_bytes || !types))) return DDT_ERR_ARG;
    for (int64_t i = 0; i < count; i++)
        if (blocklens[i] < 0 || !types[i]) return DDT_ERR_ARG;
    auto* t = new ddt_type_s();
    t->kind = T_STRUCT;
    t->blocklens.assign(blocklens, blocklens + count);
    t->displs.assign(displs_bytes, displs_bytes + count);
    t->types.assign(types, types + count);
    for (auto* k : t->types) type_retain(k);
    derive_struct(t);
    *out = t;
    return DDT_OK;
}

ddt_status_t ddt_create_resized(ddt_type_t old, int64_t lb, int64_t extent, ddt_type_t* out) {
    if (!out || !old || extent < 0) return DDT_ERR_ARG;
    auto* t = new_derived(T_RESIZED, old);
    t->size = old->size;
    t->nonempty = old->nonempty;
    t->align = old->align;
    t->sticky = true;  // explicit lb / ub markers (MPI-3.1 §4.1.7)
    t->lb = lb;
    t->ub = lb + extent;
    t->true_lb = old->true_lb;
    t->true_ub = old->true_ub;
    t->has_form = old->has_form;  // entries do not move, only the bounds
    t->form = old->form;
    *out = t;
    return DDT_OK;
}

ddt_status_t ddt_free(ddt_type_t* t) {
    if (!t) return DDT_ERR_ARG;
    if (*t) type_release(*t);
    *t = nullptr;
    return DDT_OK;
}

ddt_status_t ddt_get_size(ddt_type_t t, int64_t* size) {
    if (!t || !size) return DDT_ERR_ARG;
    *size = t->size;
    return DDT_OK;
}

ddt_status_t ddt_get_extent(ddt_type_t t, int64_t* lb, int64_t* extent) {
    if (!t || !lb || !extent) return DDT_ERR_ARG;
    *lb = t->lb;
    *extent = t->ub - t->lb;
    return DDT_OK;
}

ddt_status_t ddt_get_true_extent(ddt_type_t t, int64_t* true_lb, int64_t* true_extent) {
    if (!t || !true_lb || !true_extent) return DDT_ERR_ARG;
    *true_lb = t->true_lb;
    *true_extent = t->true_ub - t->true_lb;
    return DDT_OK;
}

}  // extern "C"

// ================================================================ flatten
namespace ddt {

// Emit the contiguous pieces of `t` placed at `base`, in typemap order.
template <class F>
static void emit_form(const Form& f, int64_t base, F&& emit) {
    const size_t D = f.dims.size();
    if (D == 0) {
        emit(base + f.base, f.seg_len);
        return;
    }
    std::vector<int64_t> idx(D, 0);
    int64_t n = f.num_segments();
    for (int64_t s = 0; s < n; s++) {
        int64_t off = base + f.base;
        for (size_t d = 0; d < D; d++) off += idx[d] * f.dims[d].stride;
        emit(off, f.seg_len);
        for (size_t d = D; d-- > 0;) {
            if (++idx[d] < f.dims[d].n) break;
            idx[d] = 0;
        }
    }
}

template <class F>
static void enumerate(const ddt_type_s* t, int64_t base, F&& emit) {
    if (!t->nonempty) return;
    if (t->has_form) {
        emit_form(t->form, base, emit);
        return;
    }
    const ddt_type_s* o = t->old;  // null for struct (per-block oldtypes)
    int64_t E = o ? type_extent(o) : 0;
    auto copy = [&](int64_t d) { enumerate(o, base + d, emit); };
    switch (t->kind) {
    case T_CONTIG:
        for (int64_t i = 0; i < t->count; i++) copy(i * E);
        break;
    case T_VECTOR:
    case T_HVECTOR: {
        int64_t S = t->kind == T_VECTOR ? t->stride * E : t->stride;
        for (int64_t i = 0; i < t->count; i++)
            for (int64_t j = 0; j < t->blocklen; j++) copy(i * S + j * E);
        break;
    }
    case T_INDEXED:
    case T_HINDEXED:
        for (size_t i = 0; i < t->blocklens.size(); i++) {
            int64_t B = t->blocklens[i];
            if (B <= 0) continue;
            int64_t d = t->kind == T_INDEXED ? t->displs[i] * E : t->displs[i];
            if (o->has_form) {
                // one block = B copies of old at d + j*E: a strided form
                Form f;
                f.base = d + o->form.base;
                f.seg_len = o->form.seg_len;
                f.dims.push_back({B, E});
                f.dims.insert(f.dims.end(), o->form.dims.begin(), o->form.dims.end());
                if (normalize(f)) emit_form(f, base, emit);
            } else {
                for (int64_t j = 0; j < B; j++) copy(d + j * E);
            }
        }
        break;
    case T_RESIZED:
        enumerate(o, base, emit);
        break;
    case T_STRUCT:
        for (size_t i = 0; i < t->blocklens.size(); i++) {
            const ddt_type_s* k = t->types[i];
            int64_t B = t->blocklens[i], Ek = type_extent(k);
            if (B <= 0 || !k->nonempty) continue;
            if (k->has_form) {
                Form f;
                f.base = t->displs[i] + k->form.base;
                f.seg_len = k->form.seg_len;
                f.dims.push_back({B, Ek});
                f.dims.insert(f.dims.end(), k->form.dims.begin(), k->form.dims.end());
                if (normalize(f)) emit_form(f, base, emit);
            } else {
                for (int64_t j = 0; j < B; j++) enumerate(k, base + t->displs[i] + j * Ek, emit);
            }
        }
        break;
    case T_SUBARRAY: {
        int nd = t->ndims;
        std::vector<int64_t> mult(nd), idx(nd, 0);
        int64_t total = 1;
        for (int k = 0; k < nd; k++) {
            int64_t m = 1;
            if (t->order == DDT_ORDER_C) {
                for (int q = k + 1; q < nd; q++) m *= t->sizes[q];
            } else {
                for (int q = 0; q < k; q++) m *= t->sizes[q];
            }
            mult[k] = m * E;
            total *= t->subsizes[k];
        }
        for (int64_t n = 0; n < total; n++) {
            int64_t d = 0;
            for (int k = 0; k < nd; k++) d += (t->starts[k] + idx[k]) * mult[k];
            copy(d);
            if (t->order == DDT_ORDER_C) {
                for (int k = nd - 1; k >= 0; k--) {
                    if (++idx[k] < t->subsizes[k]) break;
                    idx[k] = 0;
                }
            } else {
                for (int k = 0; k < nd; k++) {
                    if (++idx[k] < t->subsizes[k]) break;
                    idx[k] = 0;
                }
            }
        }
        break;
    }
    default:
        break;
    }
}

static bool segs_overlap(std::vector<Seg> v) {
    std::sort(v.begin(), v.end(), [](const Seg& a, const Seg& b) { return a.off < b.off; });
    for (size_t i = 1; i < v.size(); i++)
        if (v[i - 1].off + v[i - 1].len > v[i].off) return true;
    return false;
}

static bool form_overlaps(const Form& f) {
    // sufficient non-overlap test: sorted by |stride|, each stride clears the
    // span of everything finer; otherwise enumerate (bounded) and sort.
    std::vector<Dim> d = f.dims;
    std::sort(d.begin(), d.end(), [](const Dim& a, const Dim& b) { return uabs(a.stride) < uabs(b.stride); });
    int64_t span = f.seg_len;
    bool ok = true;
    for (auto& x : d) {
        if ((int64_t)uabs(x.stride) < span) { ok = false; break; }
        span += (x.n - 1) * (int64_t)uabs(x.stride);
    }
    if (ok) return false;
    int64_t n = f.num_segments();
    if (n > (int64_t)1 << 24) return true;  // too large to prove: conservative
    std::vector<Seg> v;
    v.reserve((size_t)n);
    emit_form(f, 0, [&](int64_t o, int64_t l) { v.push_back({o, l}); });
    return segs_overlap(v);
}

static ddt_status_t flatten(ddt_type_s* t) {
    Layout L;
    if (!t->nonempty || t->size == 0) {
        L.kind = DDT_LAYOUT_EMPTY;
        t->layout = L;
        return DDT_OK;
    }
    if (t->has_form && t->form.dims.size() <= (size_t)kMaxDims) {
        L.kind = DDT_LAYOUT_STRIDED;
        L.form = t->form;
        L.nseg = t->form.num_segments();
        L.seg_len = t->form.seg_len;
        uint64_t acc = uabs(L.form.base) | (uint64_t)L.seg_len;
        for (auto& d : L.form.dims) acc |= uabs(d.stride);
        L.align = (int)lowbit_align(acc);
        L.overlaps = form_overlaps(L.form);
        t->layout = std::move(L);
        return DDT_OK;
    }
    // list layouts: enumerate pieces in typemap order
    std::vector<Seg> pieces;
    try {
        enumerate(t, 0, [&](int64_t o, int64_t l) { pieces.push_back({o, l}); });
    } catch (const std::bad_alloc&) {
        return DDT_ERR_NOMEM;
    }
    std::vector<Seg> merged;
    merged.reserve(pieces.size());
    for (auto& p : pieces) {
        if (!merged.empty() && merged.back().off + merged.back().len == p.off)
            merged.back().len += p.len;
        else
            merged.push_back(p);
    }
    auto uniform = [](const std::vector<Seg>& v) {
        for (auto& s : v)
            if (s.len != v[0].len) return false;
        return true;
    };
    const std::vector<Seg>* use = &merged;
    if (merged.size() == 1) {
        L.kind = DDT_LAYOUT_STRIDED;
        L.form.base = merged[0].off;
        L.form.seg_len = merged[0].len;
        L.nseg = 1;
        L.seg_len = merged[0].len;
        L.align = (int)lowbit_align(uabs(L.form.base) | (uint64_t)L.seg_len);
        L.overlaps = false;
        t->layout = std::move(L);
        return DDT_OK;
    }
    if (uniform(merged)) {
        L.kind = DDT_LAYOUT_UNIFORM_LIST;
    } else if (uniform(pieces)) {
        L.kind = DDT_LAYOUT_UNIFORM_LIST;
        use = &pieces;
    } else {
        L.kind = DDT_LAYOUT_GENERAL_LIST;
    }
    L.nseg = (int64_t)use->size();
    L.seg_len = (*use)[0].len;
    uint64_t acc = 0;
    bool fits32 = true;
    L.offsets.resize(use->size());
    for (size_t i = 0; i < use->size(); i++) {
        int64_t o = (*use)[i].off;
        L.offsets[i] = o;
        acc |= uabs(o) | (uint64_t)(*use)[i].len;
        if (o < INT32_MIN || o > INT32_MAX) fits32 = false;
    }
    L.off32 = fits32;
    if (L.kind == DDT_LAYOUT_GENERAL_LIST) {
        L.lens.resize(use->size());
        L.prefix.resize(use->size() + 1);
        int64_t p = 0;
        for (size_t i = 0; i < use->size(); i++) {
            L.lens[i] = (*use)[i].len;
            L.prefix[i] = p;
            p += (*use)[i].len;
        }
        L.prefix[use->size()] = p;
    }
    L.align = (int)lowbit_align(acc);
    L.overlaps = segs_overlap(*use);
    t->layout = std::move(L);
    return DDT_OK;
}

// Do `count` instances (instance k at k*extent) write any byte twice?  Within
// one instance: the commit-time flag.  Across instances: impossible unless the
// entries span more than the extent (only resized types can), then checked
// exactly on the enumerated segments (bounded), else conservatively "yes".
bool instances_overlap(ddt_type_s* t, int64_t count) {
    if (t->layout.overlaps) return true;
    if (count <= 1 || !t->nonempty) return false;
    const int64_t ext = type_extent(t);
    if (ext >= t->true_ub - t->true_lb) return false;
    if (ext == 0) return true;  // every instance lands on the same bytes
    std::vector<Seg> one;
    enumerate(t, 0, [&](int64_t o, int64_t l) { one.push_back({o, l}); });
    if ((int64_t)one.size() * count > ((int64_t)1 << 24)) return true;
    std::vector<Seg> all;
    all.reserve(one.size() * (size_t)count);
    for (int64_t k = 0; k < count; k++)
        for (const Seg& x : one) all.push_back({x.off + k * ext, x.len});
    return segs_overlap(all);
}

ddt_status_t type_device_layout(ddt_type_s* t, int device, DeviceLayout** out) {
    // strided layouts carry everything in the descriptor: nothing to upload
    static DeviceLayout none;
    if (t->layout.kind == DDT_LAYOUT_STRIDED || t->layout.kind == DDT_LAYOUT_EMPTY) {
        *out = &none;
        return DDT_OK;
    }
    if (t->fast_dev.load(std::memory_order_acquire) == device) {
        *out = t->fast_dl.load(std::memory_order_acquire);
        if (*out) return DDT_OK;
    }
    std::lock_guard<std::mutex> g(t->mu);
    auto it = t->dev.find(device);
    if (it != t->dev.end()) {
        *out = &it->second;
        t->fast_dl.store(&it->second, std::memory_order_release);
        t->fast_dev.store(device, std::memory_order_release);
        return DDT_OK;
    }
    int prev_dev = -1;  // uploads go to `device` (callers may run with another current device)
    cudaGetDevice(&prev_dev);
    if (prev_dev != device) cudaSetDevice(device);
    struct Restore {
        int d;
        ~Restore() {
            if (d >= 0) cudaSetDevice(d);
        }
    } restore{prev_dev};
    DeviceLayout dl;
    const Layout& L = t->layout;
    cudaError_t e = cudaSuccess;
    if (L.kind == DDT_LAYOUT_UNIFORM_LIST || L.kind == DDT_LAYOUT_GENERAL_LIST) {
        bool use32 = L.kind == DDT_LAYOUT_UNIFORM_LIST && L.off32;
        size_t n = L.offsets.size();
        if (use32) {
            std::vector<int32_t> o32(n);
            for (size_t i = 0; i < n; i++) o32[i] = (int32_t)L.offsets[i];
            e = cudaMalloc(&dl.offsets, n * 4);
            if (e == cudaSuccess) e = cudaMemcpy(dl.offsets, o32.data(), n * 4, cudaMemcpyHostToDevice);
        } else {
            e = cudaMalloc(&dl.offsets, n * 8);
            if (e == cudaSuccess) e = cudaMemcpy(dl.offsets, L.offsets.data(), n * 8, cudaMemcpyHostToDevice);
        }
        if (e == cudaSuccess && L.kind == DDT_LAYOUT_GENERAL_LIST) {
            e = cudaMalloc(&dl.lens, n * 8);
            if (e == cudaSuccess) e = cudaMemcpy(dl.lens, L.lens.data(), n * 8, cudaMemcpyHostToDevice);
            if (e == cudaSuccess) e = cudaMalloc(&dl.prefix, (n + 1) * 8);
            if (e == cudaSuccess)
                e = cudaMemcpy(dl.prefix, L.prefix.data(), (n + 1) * 8, cudaMemcpyHostToDevice);
            // skip[i] = segment holding packed byte i << kSkipShift (last entry: nseg - 1)
            const int64_t bytes = L.prefix[n];
            const size_t nskip = (size_t)((bytes + (1 << kSkipShift) - 1) >> kSkipShift) + 1;
            std::vector<uint32_t> skip(nskip);
            size_t j = 0;
            for (size_t i = 0; i < nskip; i++) {
                const int64_t pos = std::min<int64_t>((int64_t)i << kSkipShift, bytes - 1);
                while (j + 1 < n && L.prefix[j + 1] <= pos) j++;
                skip[i] = (uint32_t)j;
            }
            if (e == cudaSuccess) e = cudaMalloc(&dl.skip, nskip * 4);
            if (e == cudaSuccess) e = cudaMemcpy(dl.skip, skip.data(), nskip * 4, cudaMemcpyHostToDevice);
        }
        if (e != cudaSuccess) {
            cudaFree(dl.offsets);
            cudaFree(dl.lens);
            cudaFree(dl.prefix);
            cudaFree(dl.skip);
            return cuda_fail("layout cache upload", e);
        }
    }
    auto r = t->dev.emplace(device, dl);
    *out = &r.first->second;
    t->fast_dl.store(&r.first->second, std::memory_order_release);
    t->fast_dev.store(device, std::memory_order_release);
    return DDT_OK;
}

}  // namespace ddt

extern "C" {

ddt_status_t ddt_commit(ddt_type_t t) {
    if (!t) return DDT_ERR_ARG;
    {
        std::lock_guard<std::mutex> g(t->mu);
        if (!t->committed) {
            ddt_status_t s = flatten(t);
            if (s != DDT_OK) return s;
            t->committed = true;
        }
    }
    // upload to the current device if there is one (else lazily at enqueue)
    int dev = -1;
    if (cudaGetDevice(&dev) == cudaSuccess && dev >= 0) {
        int n = 0;
        if (cudaGetDeviceCount(&n) == cudaSuccess && n > 0) {
            DeviceLayout* dl = nullptr;
            return type_device_layout(t, dev, &dl);
        }
    }
    cudaGetLastError();  // clear "no device" on CPU-only hosts
    return DDT_OK;
}

ddt_status_t ddt_get_num_segments(ddt_type_t t, int64_t* nseg) {
    if (!t || !nseg) return DDT_ERR_ARG;
    if (!t->committed) return DDT_ERR_STATE;
    *nseg = t->layout.nseg;
    return DDT_OK;
}

ddt_status_t ddt_get_layout_kind(ddt_type_t t, int32_t* kind) {
    if (!t || !kind) return DDT_ERR_ARG;
    if (!t->committed) return DDT_ERR_STATE;
    *kind = t->layout.kind;
    return DDT_OK;
}

ddt_status_t ddt_get_overlaps(ddt_type_t t, int32_t* overlaps) {
    if (!t || !overlaps) return DDT_ERR_ARG;
    if (!t->committed) return DDT_ERR_STATE;
    *overlaps = t->layout.overlaps ? 1 : 0;
    return DDT_OK;
}

ddt_status_t ddt_get_segments(ddt_type_t t, int64_t* offsets, int64_t* lengths, int64_t cap, int64_t* n) {
    if (!t || !n || cap < 0 || (cap > 0 && (!offsets || !lengths))) return DDT_ERR_ARG;
    if (!t->committed) return DDT_ERR_STATE;
    const Layout& L = t->layout;
    *n = L.nseg;
    int64_t i = 0;
    if (L.kind == DDT_LAYOUT_STRIDED) {
        emit_form(L.form, 0, [&](int64_t o, int64_t l) {
            if (i < cap) { offsets[i] = o; lengths[i] = l; }
            i++;
        });
    } else if (L.kind != DDT_LAYOUT_EMPTY) {
        for (; i < L.nseg && i < cap; i++) {
            offsets[i] = L.offsets[i];
            lengths[i] = L.kind == DDT_LAYOUT_GENERAL_LIST ? L.lens[i] : L.seg_len;
        }
    }
    return DDT_OK;
}

const char* ddt_strerror(ddt_status_t s) {
    switch (s) {
    case DDT_OK: return "ok";
    case DDT_ERR_ARG: return "invalid argument";
    case DDT_ERR_STATE: return "invalid state (type not committed / bad lifecycle)";
    case DDT_ERR_QUEUE_FULL: return "request list full (flush and retry)";
    case DDT_ERR_OVERLAP: return "unpack into a datatype with overlapping entries";
    case DDT_ERR_NOMEM: return "out of memory";
    case DDT_ERR_CUDA: return "CUDA error";
    case DDT_ERR_NCCL: return "NCCL error";
    case DDT_ERR_SIZE_MISMATCH: return "matched send/recv sizes differ";
    case DDT_ERR_TIMEOUT: return "device wait timed out";
    case DDT_ERR_UNSUPPORTED: return "unsupported";
    case DDT_ERR_NODEV: return "no CUDA device";
    default: return "unknown error";
    }
}

const char* ddt_last_error_message(void) { return ddt::last_error(); }
int32_t ddt_version(void) { return 100; }

}  // extern "C"
