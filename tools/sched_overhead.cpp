// sched_overhead.cpp -- host-side cost of the request list + scheduler
// (§IV-A, Fig 11: "scheduling overhead ... as low as 2 us per
// message"), measured through the C ABI with no Python in the loop.
// Build + run on a GPU box:  tools/sched_overhead.sh
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "ddt.h"

static double now_ns() {
    return (double)std::chrono::duration_cast<std::chrono::nanoseconds>(
               std::chrono::steady_clock::now().time_since_epoch())
        .count();
}

#define CHECK(x)                                                            \
    do {                                                                    \
        long long _r = (long long)(x);                                      \
        if (_r < 0) {                                                       \
            fprintf(stderr, "%s -> %lld (%s)\n", #x, _r, ddt_last_error_message()); \
            return 1;                                                       \
        }                                                                   \
    } while (0)

int main() {
    cudaStream_t s;
    cudaSetDevice(0);
    cudaStreamCreate(&s);
    ddt_queue_t q;
    CHECK(ddt_queue_create(0, s, 8192, &q));
    ddt_type_t dbl, vec, sub;
    CHECK(ddt_type_basic(DDT_DOUBLE, &dbl));
    CHECK(ddt_create_vector(4, 32, 64, dbl, &vec));  // 1 KiB, 256 B blocks (configs[4] layout)
    CHECK(ddt_commit(vec));
    int64_t sizes[3] = {130, 130, 130}, subs[3] = {128, 128, 1}, starts[3] = {1, 1, 128};
    CHECK(ddt_create_subarray(3, sizes, subs, starts, DDT_ORDER_C, dbl, &sub));  // a configs[1] x-face
    CHECK(ddt_commit(sub));
    const int N = 4096;
    char *src, *dst;
    cudaMalloc(&src, (size_t)N * 2048);
    cudaMalloc(&dst, (size_t)N * 1024);
    // warm up
    for (int i = 0; i < 64; i++) CHECK(ddt_pack_enqueue(q, vec, src + 2048 * i, 1, dst + 1024 * i));
    CHECK(ddt_wait(q));

    double t0 = now_ns();
    for (int i = 0; i < N; i++) CHECK(ddt_pack_enqueue(q, vec, src + 2048 * (i % N), 1, dst + 1024 * (i % N)));
    double t1 = now_ns();
    CHECK(ddt_flush(q));
    double t2 = now_ns();
    CHECK(ddt_wait(q));
    double enq_vec = (t1 - t0) / N, flush_big = (t2 - t1) / 1e3;

    char* arr;
    cudaMalloc(&arr, (size_t)130 * 130 * 130 * 8);
    t0 = now_ns();
    for (int i = 0; i < 1024; i++) CHECK(ddt_pack_enqueue(q, sub, arr, 1, dst + 131072 * (i % 8)));
    t1 = now_ns();
    CHECK(ddt_wait(q));
    double enq_sub = (t1 - t0) / 1024;

    // enqueue + flush cycles at several batch sizes (host time per request)
    printf("{\"enqueue_ns_vector\": %.1f, \"enqueue_ns_subarray_face\": %.1f, \"flush_us_4096_requests\": %.2f",
           enq_vec, enq_sub, flush_big);
    for (int B : {1, 8, 32, 64, 256, 1024}) {
        const int reps = 2000 / B + 5;
        t0 = now_ns();
        for (int r = 0; r < reps; r++) {
            for (int i = 0; i < B; i++) CHECK(ddt_pack_enqueue(q, vec, src + 2048 * i, 1, dst + 1024 * i));
            CHECK(ddt_flush(q));
        }
        t1 = now_ns();
        CHECK(ddt_wait(q));
        printf(", \"host_us_per_request_B%d\": %.3f", B, (t1 - t0) / 1e3 / (reps * B));
    }
    printf("}\n");
    ddt_queue_destroy(q);
    return 0;
}
