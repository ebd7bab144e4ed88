/*
 * ddt_oracle.c -- TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
 * reference for MPI derived-datatype pack / unpack.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  The product path
 * (paper_conf_cluster_chukzsp20_b200/) never links, imports or calls it, and this
 * file shares no code, header, table or helper with the product.
 *
 * What it computes:
 *   - The paper's method computes exactly MPI_Pack / MPI_Unpack of a
 *     derived datatype, only faster (§II-B P:81 "MPI standard defines various
 *     derived datatypes including vector, indexed, subarray, struct";
 *     §III-A Alg 1 P:98-119 MPI_Pack/MPI_Unpack; §IV-A.1 P:189-197 the
 *     request's "data layout").  Datatype semantics are deferred by the paper
 *     to the MPI standard [29]: typemaps, MPI-3.1 §4.1.
 *   - So the oracle is the plain definition written out: a recursive walk of
 *     the constructor tree in TYPEMAP ORDER, one basic element at a time,
 *     memcpy'ing each element.
 *
 * Definitions followed (MPI-3.1 §4.1, restated, not pasted):
 *   vector(c,b,s,old):  for i<c, for j<b: copy of old at (i*s + j)*ext(old)
 *   hvector(c,b,S,old): for i<c, for j<b: copy of old at i*S + j*ext(old)
 *   indexed(n,B,D,old): for i<n, for j<B[i]: copy of old at (D[i]+j)*ext(old)
 *   hindexed(n,B,D,old):for i<n, for j<B[i]: copy of old at D[i] + j*ext(old)
 *   contiguous(n,old):  for i<n: copy of old at i*ext(old)
 *   struct(n,B,D,T[]):  for i<n, for j<B[i]: copy of T[i] at D[i] + j*ext(T[i])
 *                       (byte displacements).  ub carries the alignment
 *                       increment epsilon (MPI-3.1 §4.1, "ub(Typemap) = max_j
 *                       (disp_j + sizeof(type_j)) + epsilon", epsilon = the
 *                       least non-negative increment that rounds the extent to
 *                       a multiple of max_i k_i, k_i = alignment of basic type
 *                       i = its size here) unless the typemap carries explicit
 *                       bounds markers (a resized or subarray type beneath it,
 *                       MPI-3.1 §4.1.6-4.1.7).  DESIGN.md reading R2.
 *   resized(old,lb,ex): the typemap of old with lb / extent set to (lb, ex)
 *                       (MPI-3.1 §4.1.7); true bounds stay those of the entries
 *   subarray(nd,sizes,subsizes,starts,order,old): C order = dim 0 outermost,
 *     last dim fastest; Fortran = dim nd-1 outermost, dim 0 fastest; element
 *     (i_0..i_{nd-1}) is a copy of old at
 *     sum_k (starts[k]+i_k) * (prod of sizes of the faster dims) * ext(old);
 *     the result is resized to lb = 0, extent = prod(sizes)*ext(old)
 *     (MPI-3.1 §4.1.3).
 *   lb / ub: min / max over every placed (non-empty) copy of the oldtype of
 *     copy_disp + lb(old) / copy_disp + ub(old); basic: [0, sizeof).  Empty
 *     type: lb = ub = 0 (reading R3).  Alignment epsilon: struct
 *     only (R2, see above); k is found by enumerating the struct's entries.
 *   true lb / ub: min / max over the actual basic entries.
 *   pack(src,count,T,out): instance k at k*extent(T); entries copied in
 *     typemap order to consecutive packed positions (R1, R8, R9).
 *   unpack: the same walk with the copy direction reversed.
 *
 * Every quantity is derived by ENUMERATION (walking the tree), never by the
 * closed forms the product library uses, so the two pin each other.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { OK_BASIC = 0, OK_CONTIG, OK_VECTOR, OK_HVECTOR, OK_INDEXED, OK_HINDEXED, OK_SUBARRAY, OK_STRUCT, OK_RESIZED };

typedef struct orc_type {
    int kind;
    int64_t elem_size;              /* basic only */
    int64_t count, blocklen, stride; /* contig / vector / hvector */
    int64_t nblocks;
    int64_t *blocklens, *displs;    /* indexed / hindexed */
    int ndims, order;
    int64_t sizes[16], subsizes[16], starts[16];
    struct orc_type *old;
    struct orc_type **types;        /* struct: one oldtype per block */
    int64_t rlb, rextent;           /* resized */
} orc_type;

/* ---------------------------------------------------------------- builders */

static orc_type *orc_new(int kind) {
    orc_type *t = (orc_type *)calloc(1, sizeof(orc_type));
    t->kind = kind;
    return t;
}

orc_type *orc_basic(int64_t elem_size) {
    orc_type *t = orc_new(OK_BASIC);
    t->elem_size = elem_size;
    return t;
}

orc_type *orc_contiguous(int64_t count, orc_type *old) {
    orc_type *t = orc_new(OK_CONTIG);
    t->count = count;
    t->old = old;
    return t;
}

orc_type *orc_vector(int64_t count, int64_t blocklen, int64_t stride, orc_type *old) {
    orc_type *t = orc_new(OK_VECTOR);
    t->count = count; t->blocklen = blocklen; t->stride = stride; t->old = old;
    return t;
}

orc_type *orc_hvector(int64_t count, int64_t blocklen, int64_t stride_bytes, orc_type *old) {
    orc_type *t = orc_new(OK_HVECTOR);
    t->count = count; t->blocklen = blocklen; t->stride = stride_bytes; t->old = old;
    return t;
}

static orc_type *orc_blocks(int kind, int64_t n, const int64_t *bl, const int64_t *d, orc_type *old) {
    orc_type *t = orc_new(kind);
    t->nblocks = n;
    t->blocklens = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    t->displs = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; i++) { t->blocklens[i] = bl[i]; t->displs[i] = d[i]; }
    t->old = old;
    return t;
}

orc_type *orc_indexed(int64_t n, const int64_t *bl, const int64_t *displs, orc_type *old) {
    return orc_blocks(OK_INDEXED, n, bl, displs, old);
}

orc_type *orc_hindexed(int64_t n, const int64_t *bl, const int64_t *displs_bytes, orc_type *old) {
    return orc_blocks(OK_HINDEXED, n, bl, displs_bytes, old);
}

orc_type *orc_subarray(int ndims, const int64_t *sizes, const int64_t *subsizes,
                       const int64_t *starts, int order /*0=C,1=Fortran*/, orc_type *old) {
    if (ndims < 1 || ndims > 16) return NULL;
    orc_type *t = orc_new(OK_SUBARRAY);
    t->ndims = ndims; t->order = order; t->old = old;
    for (int k = 0; k < ndims; k++) {
        t->sizes[k] = sizes[k]; t->subsizes[k] = subsizes[k]; t->starts[k] = starts[k];
    }
    return t;
}

orc_type *orc_struct(int64_t n, const int64_t *bl, const int64_t *displs_bytes, orc_type **types) {
    orc_type *t = orc_blocks(OK_STRUCT, n, bl, displs_bytes, NULL);
    t->types = (orc_type **)malloc(sizeof(orc_type *) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; i++) t->types[i] = types[i];
    return t;
}

orc_type *orc_resized(orc_type *old, int64_t lb, int64_t extent) {
    orc_type *t = orc_new(OK_RESIZED);
    t->old = old; t->rlb = lb; t->rextent = extent;
    return t;
}

/* The oracle never frees shared oldtypes; tests build small trees. */
void orc_free(orc_type *t) {
    if (!t) return;
    free(t->blocklens);
    free(t->displs);
    free(t->types);
    free(t);
}

/* ------------------------------------------------- walk (typemap order) */

typedef void (*orc_emit_fn)(void *ctx, int64_t disp, int64_t nbytes);

static int64_t orc_extent(const orc_type *t);

/* Visit every basic entry of T placed at byte displacement `base`, in
 * typemap order.  This is the definition of the typemap. */
static void orc_walk(const orc_type *t, int64_t base, orc_emit_fn emit, void *ctx) {
    switch (t->kind) {
    case OK_BASIC:
        emit(ctx, base, t->elem_size);
        return;
    case OK_CONTIG: {
        int64_t e = orc_extent(t->old);
        for (int64_t i = 0; i < t->count; i++) orc_walk(t->old, base + i * e, emit, ctx);
        return;
    }
    case OK_VECTOR: {
        int64_t e = orc_extent(t->old);
        for (int64_t i = 0; i < t->count; i++)
            for (int64_t j = 0; j < t->blocklen; j++)
                orc_walk(t->old, base + (i * t->stride + j) * e, emit, ctx);
        return;
    }
    case OK_HVECTOR: {
        int64_t e = orc_extent(t->old);
        for (int64_t i = 0; i < t->count; i++)
            for (int64_t j = 0; j < t->blocklen; j++)
                orc_walk(t->old, base + i * t->stride + j * e, emit, ctx);
        return;
    }
    case OK_INDEXED: {
        int64_t e = orc_extent(t->old);
        for (int64_t i = 0; i < t->nblocks; i++)
            for (int64_t j = 0; j < t->blocklens[i]; j++)
                orc_walk(t->old, base + (t->displs[i] + j) * e, emit, ctx);
        return;
    }
    case OK_HINDEXED: {
        int64_t e = orc_extent(t->old);
        for (int64_t i = 0; i < t->nblocks; i++)
            for (int64_t j = 0; j < t->blocklens[i]; j++)
                orc_walk(t->old, base + t->displs[i] + j * e, emit, ctx);
        return;
    }
    case OK_STRUCT:
        for (int64_t i = 0; i < t->nblocks; i++) {
            int64_t e = orc_extent(t->types[i]);
            for (int64_t j = 0; j < t->blocklens[i]; j++)
                orc_walk(t->types[i], base + t->displs[i] + j * e, emit, ctx);
        }
        return;
    case OK_RESIZED:
        orc_walk(t->old, base, emit, ctx);
        return;
    case OK_SUBARRAY: {
        /* Odometer over the subsizes box.  C order: last dim fastest.
         * Fortran order: dim 0 fastest. */
        int nd = t->ndims;
        int64_t e = orc_extent(t->old);
        int64_t mult[16];
        int64_t total = 1;
        for (int k = 0; k < nd; k++) {
            int64_t m = 1;
            if (t->order == 0) { for (int q = k + 1; q < nd; q++) m *= t->sizes[q]; }
            else               { for (int q = 0; q < k; q++)       m *= t->sizes[q]; }
            mult[k] = m;
            total *= t->subsizes[k];
        }
        int64_t idx[16];
        for (int k = 0; k < nd; k++) idx[k] = 0;
        for (int64_t n = 0; n < total; n++) {
            int64_t d = 0;
            for (int k = 0; k < nd; k++) d += (t->starts[k] + idx[k]) * mult[k];
            orc_walk(t->old, base + d * e, emit, ctx);
            /* advance the fastest dimension first */
            if (t->order == 0) {
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
        return;
    }
    }
}

/* ------------------------------------------------------ size, bounds */

typedef struct { int64_t n; int64_t bytes; int64_t lo, hi; } orc_acc;

static void orc_acc_emit(void *ctx, int64_t disp, int64_t nbytes) {
    orc_acc *a = (orc_acc *)ctx;
    if (a->n == 0 || disp < a->lo) a->lo = disp;
    if (a->n == 0 || disp + nbytes > a->hi) a->hi = disp + nbytes;
    a->n += 1;
    a->bytes += nbytes;
}

/* number of basic entries and their total size (enumerated) */
int64_t orc_num_entries(const orc_type *t) {
    orc_acc a = {0, 0, 0, 0};
    orc_walk(t, 0, orc_acc_emit, &a);
    return a.n;
}

int64_t orc_size(const orc_type *t) {
    orc_acc a = {0, 0, 0, 0};
    orc_walk(t, 0, orc_acc_emit, &a);
    return a.bytes;
}

/* lb / ub by enumeration over placed copies of the oldtype (MPI-3.1 §4.1).
 * Returns 0 if the type has no entries (then lb = ub = 0). */
static int orc_bounds(const orc_type *t, int64_t *lb, int64_t *ub);

typedef struct { int any; int64_t lo, hi; } orc_bacc;

static void orc_bacc_add(orc_bacc *b, int64_t lo, int64_t hi) {
    if (!b->any || lo < b->lo) b->lo = lo;
    if (!b->any || hi > b->hi) b->hi = hi;
    b->any = 1;
}

/* Explicit lb / ub markers somewhere in the tree (resized, subarray). */
static int orc_has_markers(const orc_type *t) {
    switch (t->kind) {
    case OK_BASIC: return 0;
    case OK_RESIZED: case OK_SUBARRAY: return 1;
    case OK_STRUCT:
        for (int64_t i = 0; i < t->nblocks; i++)
            if (orc_has_markers(t->types[i])) return 1;
        return 0;
    default: return orc_has_markers(t->old);
    }
}

/* max_i k_i over the basic entries of a typemap: every emitted entry is one
 * basic element whose alignment equals its size (1, 4 or 8 bytes). */
static void orc_align_emit(void *ctx, int64_t disp, int64_t nbytes) {
    (void)disp;
    int64_t *k = (int64_t *)ctx;
    if (nbytes > *k) *k = nbytes;
}

static int orc_bounds(const orc_type *t, int64_t *lb, int64_t *ub) {
    if (t->kind == OK_BASIC) { *lb = 0; *ub = t->elem_size; return 1; }
    if (t->kind == OK_SUBARRAY) {
        /* resized: lb = 0, extent = prod(sizes) * ext(old) -- if any entries */
        int64_t olb, oub;
        int64_t total = 1, prod = 1;
        for (int k = 0; k < t->ndims; k++) { total *= t->subsizes[k]; prod *= t->sizes[k]; }
        int nonempty_old = orc_bounds(t->old, &olb, &oub);
        if (total == 0 || !nonempty_old) { *lb = 0; *ub = 0; return 0; }
        *lb = 0;
        *ub = prod * (oub - olb);
        return 1;
    }
    if (t->kind == OK_RESIZED) {
        /* explicit bounds; a type without entries still contributes none (R3) */
        int64_t olb, oub;
        int nonempty_old = orc_bounds(t->old, &olb, &oub);
        *lb = t->rlb;
        *ub = t->rlb + t->rextent;
        return nonempty_old;
    }
    if (t->kind == OK_STRUCT) {
        orc_bacc b = {0, 0, 0};
        for (int64_t i = 0; i < t->nblocks; i++) {
            int64_t olb, oub;
            if (!orc_bounds(t->types[i], &olb, &oub)) continue;
            int64_t e = oub - olb;
            for (int64_t j = 0; j < t->blocklens[i]; j++) {
                int64_t d = t->displs[i] + j * e;
                orc_bacc_add(&b, d + olb, d + oub);
            }
        }
        if (!b.any) { *lb = 0; *ub = 0; return 0; }
        *lb = b.lo; *ub = b.hi;
        if (!orc_has_markers(t)) { /* epsilon: round the extent up to a multiple of k */
            int64_t k = 1;
            orc_walk(t, 0, orc_align_emit, &k);
            int64_t ext = b.hi - b.lo;
            while (ext % k != 0) ext++;
            *ub = b.lo + ext;
        }
        return 1;
    }
    int64_t olb, oub;
    int nonempty_old = orc_bounds(t->old, &olb, &oub);
    int64_t e = oub - olb;
    orc_bacc b = {0, 0, 0};
    if (nonempty_old) {
        switch (t->kind) {
        case OK_CONTIG:
            for (int64_t i = 0; i < t->count; i++) orc_bacc_add(&b, i * e + olb, i * e + oub);
            break;
        case OK_VECTOR:
            for (int64_t i = 0; i < t->count; i++)
                for (int64_t j = 0; j < t->blocklen; j++) {
                    int64_t d = (i * t->stride + j) * e;
                    orc_bacc_add(&b, d + olb, d + oub);
                }
            break;
        case OK_HVECTOR:
            for (int64_t i = 0; i < t->count; i++)
                for (int64_t j = 0; j < t->blocklen; j++) {
                    int64_t d = i * t->stride + j * e;
                    orc_bacc_add(&b, d + olb, d + oub);
                }
            break;
        case OK_INDEXED:
            for (int64_t i = 0; i < t->nblocks; i++)
                for (int64_t j = 0; j < t->blocklens[i]; j++) {
                    int64_t d = (t->displs[i] + j) * e;
                    orc_bacc_add(&b, d + olb, d + oub);
                }
            break;
        case OK_HINDEXED:
            for (int64_t i = 0; i < t->nblocks; i++)
                for (int64_t j = 0; j < t->blocklens[i]; j++) {
                    int64_t d = t->displs[i] + j * e;
                    orc_bacc_add(&b, d + olb, d + oub);
                }
            break;
        }
    }
    if (!b.any) { *lb = 0; *ub = 0; return 0; }
    *lb = b.lo; *ub = b.hi;
    return 1;
}

static int64_t orc_extent(const orc_type *t) {
    int64_t lb, ub;
    orc_bounds(t, &lb, &ub);
    return ub - lb;
}

void orc_get_extent(const orc_type *t, int64_t *lb, int64_t *extent) {
    int64_t l, u;
    orc_bounds(t, &l, &u);
    *lb = l;
    *extent = u - l;
}

void orc_get_true_extent(const orc_type *t, int64_t *true_lb, int64_t *true_extent) {
    orc_acc a = {0, 0, 0, 0};
    orc_walk(t, 0, orc_acc_emit, &a);
    if (a.n == 0) { *true_lb = 0; *true_extent = 0; return; }
    *true_lb = a.lo;
    *true_extent = a.hi - a.lo;
}

/* ---------------------------------------------------- typemap listing */

typedef struct { int64_t *disp; int64_t *len; int64_t cap, n; } orc_list;

static void orc_list_emit(void *ctx, int64_t disp, int64_t nbytes) {
    orc_list *l = (orc_list *)ctx;
    if (l->n < l->cap) { l->disp[l->n] = disp; l->len[l->n] = nbytes; }
    l->n += 1;
}

/* Writes up to cap (disp, nbytes) entries of count instances; returns the
 * total number of entries. */
int64_t orc_typemap(const orc_type *t, int64_t count, int64_t *disp, int64_t *len, int64_t cap) {
    orc_list l = {disp, len, cap, 0};
    int64_t e = orc_extent(t);
    for (int64_t k = 0; k < count; k++) orc_walk(t, k * e, orc_list_emit, &l);
    return l.n;
}

/* --------------------------------------------------------- pack/unpack */

typedef struct { const uint8_t *src; uint8_t *out; int64_t pos; } orc_pack_ctx;

static void orc_pack_emit(void *ctx, int64_t disp, int64_t nbytes) {
    orc_pack_ctx *c = (orc_pack_ctx *)ctx;
    memcpy(c->out + c->pos, c->src + disp, (size_t)nbytes);
    c->pos += nbytes;
}

typedef struct { const uint8_t *in; uint8_t *dst; int64_t pos; } orc_unpack_ctx;

static void orc_unpack_emit(void *ctx, int64_t disp, int64_t nbytes) {
    orc_unpack_ctx *c = (orc_unpack_ctx *)ctx;
    memcpy(c->dst + disp, c->in + c->pos, (size_t)nbytes);
    c->pos += nbytes;
}

/* src: the MPI buffer address (displacements are relative to it and may be
 * negative).  out: count*size bytes.  Returns bytes written. */
int64_t orc_pack(const orc_type *t, const void *src, int64_t count, void *out) {
    orc_pack_ctx c = {(const uint8_t *)src, (uint8_t *)out, 0};
    int64_t e = orc_extent(t);
    for (int64_t k = 0; k < count; k++) orc_walk(t, k * e, orc_pack_emit, &c);
    return c.pos;
}

int64_t orc_unpack(const orc_type *t, const void *in, int64_t count, void *dst) {
    orc_unpack_ctx c = {(const uint8_t *)in, (uint8_t *)dst, 0};
    int64_t e = orc_extent(t);
    for (int64_t k = 0; k < count; k++) orc_walk(t, k * e, orc_unpack_emit, &c);
    return c.pos;
}
