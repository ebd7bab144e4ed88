/* abi_smoke.c -- the C ABI used from plain C99 (no Python, no torch): build a
 * configs[0] vector type and a subarray face, pack + unpack through one queue,
 * query the request states, and check the bytes against the MPI definition
 * spelled out for these two fixed types (a smoke test of the boundary; the
 * parity proper is tests/test_gpu_parity.py against the oracle). */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <cuda_runtime.h>

#include "ddt.h"

#define CK(x)                                                                            \
    do {                                                                                 \
        long long r_ = (long long)(x);                                                   \
        if (r_ < 0) {                                                                    \
            fprintf(stderr, "FAIL %s -> %lld %s\n", #x, r_, ddt_last_error_message());   \
            return 1;                                                                    \
        }                                                                                \
    } while (0)

int main(void) {
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        printf("SKIP no device\n");
        return 0;
    }
    ddt_type_t dbl, vec, face;
    CK(ddt_type_basic(DDT_DOUBLE, &dbl));
    CK(ddt_create_vector(16, 4, 64, dbl, &vec)); /* BASELINE configs[0] */
    CK(ddt_commit(vec));
    int64_t size = 0, lb = 0, ext = 0;
    CK(ddt_get_size(vec, &size));
    CK(ddt_get_extent(vec, &lb, &ext));
    if (size != 512 || lb != 0 || ext != 7712) { fprintf(stderr, "FAIL closed forms\n"); return 1; }
    int64_t sizes[3] = {10, 12, 14}, subs[3] = {8, 10, 1}, starts[3] = {1, 1, 12};
    CK(ddt_create_subarray(3, sizes, subs, starts, DDT_ORDER_C, dbl, &face));
    CK(ddt_commit(face));

    const size_t n = 10 * 12 * 14;
    double* h_src = malloc(8 * 1000);
    double* h_arr = malloc(8 * n);
    for (int i = 0; i < 1000; i++) h_src[i] = (double)i;
    for (size_t i = 0; i < n; i++) h_arr[i] = -(double)i;
    double *d_src, *d_pk, *d_back, *d_arr, *d_fpk;
    cudaMalloc((void**)&d_src, 8 * 1000);
    cudaMalloc((void**)&d_pk, 512);
    cudaMalloc((void**)&d_back, 8 * 1000);
    cudaMalloc((void**)&d_arr, 8 * n);
    cudaMalloc((void**)&d_fpk, 8 * 80);
    cudaMemcpy(d_src, h_src, 8 * 1000, cudaMemcpyHostToDevice);
    cudaMemcpy(d_arr, h_arr, 8 * n, cudaMemcpyHostToDevice);
    cudaMemset(d_back, 0, 8 * 1000);

    ddt_queue_t q;
    CK(ddt_queue_create(0, NULL, 0, &q));
    int64_t u0 = ddt_pack_enqueue(q, vec, d_src, 1, d_pk);
    int64_t u1 = ddt_pack_enqueue(q, face, d_arr, 1, d_fpk);
    CK(u0);
    CK(u1);
    int32_t st = -1;
    CK(ddt_query(q, u0, &st));
    if (st != DDT_PENDING) { fprintf(stderr, "FAIL state before flush %d\n", st); return 1; }
    if (ddt_flush(q) != 2) { fprintf(stderr, "FAIL flush count\n"); return 1; }
    CK(ddt_unpack_enqueue(q, vec, d_pk, 1, d_back));
    CK(ddt_wait(q));
    CK(ddt_query(q, u1, &st));
    if (st != DDT_COMPLETED) { fprintf(stderr, "FAIL state after wait %d\n", st); return 1; }

    double pk[64], fpk[80], back[1000];
    cudaMemcpy(pk, d_pk, 512, cudaMemcpyDeviceToHost);
    cudaMemcpy(fpk, d_fpk, 640, cudaMemcpyDeviceToHost);
    cudaMemcpy(back, d_back, 8000, cudaMemcpyDeviceToHost);
    for (int i = 0; i < 16; i++)
        for (int j = 0; j < 4; j++)
            if (pk[4 * i + j] != (double)(64 * i + j)) { fprintf(stderr, "FAIL vector pack\n"); return 1; }
    for (int k = 0; k < 1000; k++) {
        int in_block = (k % 64) < 4 && k < 15 * 64 + 4;
        if (back[k] != (in_block ? (double)k : 0.0)) { fprintf(stderr, "FAIL vector unpack at %d\n", k); return 1; }
    }
    int p = 0;
    for (int z = 1; z < 9; z++)
        for (int y = 1; y < 11; y++)
            if (fpk[p++] != -(double)((z * 12 + y) * 14 + 12)) { fprintf(stderr, "FAIL face pack\n"); return 1; }
    ddt_queue_stats_t s;
    CK(ddt_queue_get_stats(q, &s));
    if (s.launches != 2 || s.requests != 3) { fprintf(stderr, "FAIL stats\n"); return 1; }
    CK(ddt_queue_destroy(q));
    CK(ddt_free(&vec));
    CK(ddt_free(&face));
    printf("OK abi_smoke (C99): vector + subarray face pack/unpack, states, stats\n");
    return 0;
}
