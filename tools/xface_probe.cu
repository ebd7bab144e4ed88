// xface_probe.cu -- diagnostic: how fast can B200 DRAM serve the 8-B x-face
// halo pattern (one double per 4112-B row of a 514^3 C-order array, the
// configs[3] COMB x-faces), and does the order in which the four accesses of a
// row (read col 1, read col 512, write col 513, write col 0 -- the P = 1
// periodic self exchange) are issued matter?  Thread per (row, access group);
// CUDA-event timed after an L2 flush (write + read of 512 MiB, so the L2 holds
// clean lines), median of 7.  Prints one JSON line per variant.
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <algorithm>

constexpr long long N = 514;           // 512 interior + 2 ghosts
constexpr long long R = 512 * 512;     // interior rows
__device__ __forceinline__ long long row_base(long long r) { return (((r / 512) + 1) * N + (r % 512) + 1) * N; }

__global__ void pack1(const double* __restrict__ a, double* o1) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < R) o1[i] = a[row_base(i) + 1];
}
__global__ void pack2(const double* __restrict__ a, double* o1, double* o2) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < R) { long long b = row_base(i); o1[i] = a[b + 1]; o2[i] = a[b + 512]; }
}
// one column, U rows per thread (rows i, i + R/U, ...): the memory-level parallelism of pack2 / our ub
template <int U>
__global__ void pack1_u(const double* __restrict__ a, double* o1) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= R / U) return;
    double t[U];
#pragma unroll
    for (int u = 0; u < U; u++) t[u] = a[row_base(i + u * (R / U)) + 1];
#pragma unroll
    for (int u = 0; u < U; u++) o1[i + u * (R / U)] = t[u];
}
// two packs (col 1 -> o1, col 512 -> o2) as two requests, items of C rows: split (C = R) or interleaved
template <long long C>
__global__ void pack2_chunked(const double* __restrict__ a, double* o1, double* o2) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= 2 * R) return;
    long long chunk = i / C, m = chunk & 1, r = (chunk >> 1) * C + i % C;
    if (m == 0) o1[r] = a[row_base(r) + 1];
    else o2[r] = a[row_base(r) + 512];
}
__global__ void pack2_split(const double* __restrict__ a, double* o1, double* o2) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < R) o1[i] = a[row_base(i) + 1];
    else if (i < 2 * R) o2[i - R] = a[row_base(i - R) + 512];
}
__global__ void write1(double* a) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < R) a[row_base(i)] = 1.0;
}
// every access of a row by one thread
__global__ void self_fused(double* a) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < R) { long long b = row_base(i); double t1 = a[b + 1], t2 = a[b + 512]; a[b + 513] = t1; a[b] = t2; }
}
// message -x over all rows, then message +x over all rows (one launch, threads in order)
__global__ void self_split(double* a) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < R) { long long b = row_base(i); a[b + 513] = a[b + 1]; }
    else if (i < 2 * R) { long long b = row_base(i - R); a[b] = a[b + 512]; }
}
// messages interleaved in chunks of C rows (an item-level interleave of the two requests)
template <int C>
__global__ void self_chunked(double* a) {
    long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= 2 * R) return;
    long long chunk = i / C, m = chunk & 1, r = (chunk >> 1) * C + i % C;
    long long b = row_base(r);
    if (m == 0) a[b + 513] = a[b + 1];
    else a[b] = a[b + 512];
}
__global__ void fill(unsigned* p, long long n, unsigned v) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) p[i] = v;
}
__global__ void sum(const unsigned* p, long long n, unsigned* out) {
    unsigned s = 0;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) s += p[i];
    if (s == 0x12345678u) *out = s;
}

int main() {
    double* a;
    double *o1, *o2;
    unsigned *fl, *junk;
    const long long nflush = (512ll << 20) / 4;
    cudaMalloc(&a, N * N * N * 8);
    cudaMalloc(&o1, R * 8);
    cudaMalloc(&o2, R * 8);
    cudaMalloc(&fl, nflush * 4);
    cudaMalloc(&junk, 64);
    cudaMemset(a, 0, N * N * N * 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto run = [&](const char* name, int accesses, auto launch, bool clean) {
        std::vector<float> t;
        for (int rep = 0; rep < 8; rep++) {
            fill<<<1184, 256>>>(fl, nflush, rep);
            if (clean) sum<<<1184, 256>>>(fl, nflush, junk);
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (rep) t.push_back(ms * 1e3f);
        }
        std::sort(t.begin(), t.end());
        float us = t[t.size() / 2];
        // 8 B per access of useful payload; 64 B per access at the DRAM's scattered granularity
        printf("{\"variant\": \"%s\", \"l2\": \"%s\", \"us\": %.2f, \"accesses\": %lld, \"G_access_per_s\": %.2f, \"payload_GBs\": %.1f, \"dram64_GBs\": %.1f}\n",
               name, clean ? "clean" : "dirty", us, (long long)accesses * R, accesses * R / us / 1e3,
               accesses * R * 8.0 / us / 1e3, accesses * R * 64.0 / us / 1e3);
    };
    const int T = 256;
    const long long B1 = (R + T - 1) / T, B2 = (2 * R + T - 1) / T;
    for (int clean = 1; clean >= 0; clean--) {
        run("pack_col1", 2, [&] { pack1<<<B1, T>>>(a, o1); }, clean);
        run("pack_col1_col512", 4, [&] { pack2<<<B1, T>>>(a, o1, o2); }, clean);
        run("pack_col1_2rows_per_thread", 2, [&] { pack1_u<2><<<(R / 2 + T - 1) / T, T>>>(a, o1); }, clean);
        run("pack_col1_4rows_per_thread", 2, [&] { pack1_u<4><<<(R / 4 + T - 1) / T, T>>>(a, o1); }, clean);
        run("pack2_split_messages", 4, [&] { pack2_split<<<B2, T>>>(a, o1, o2); }, clean);
        run("pack2_chunked_1024", 4, [&] { pack2_chunked<1024><<<B2, T>>>(a, o1, o2); }, clean);
        run("pack2_chunked_32", 4, [&] { pack2_chunked<32><<<B2, T>>>(a, o1, o2); }, clean);
        run("write_col0_only", 1, [&] { write1<<<B1, T>>>(a); }, clean);
        run("self_fused_per_row", 4, [&] { self_fused<<<B1, T>>>(a); }, clean);
        run("self_split_messages", 4, [&] { self_split<<<B2, T>>>(a); }, clean);
        run("self_chunked_1024", 4, [&] { self_chunked<1024><<<B2, T>>>(a); }, clean);
        run("self_chunked_8192", 4, [&] { self_chunked<8192><<<B2, T>>>(a); }, clean);
        run("self_chunked_32", 4, [&] { self_chunked<32><<<B2, T>>>(a); }, clean);
    }
    cudaError_t err = cudaDeviceSynchronize();
    if (err != cudaSuccess) { printf("{\"error\": \"%s\"}\n", cudaGetErrorString(err)); return 1; }
    return 0;
}
