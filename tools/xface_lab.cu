// xface_lab.cu -- diagnostic: schedules for the COMB x faces (configs[3] P = 1,
// four 514^3 double arrays; per interior row (z, y) the periodic self exchange
// moves cell 512 -> ghost 0 and cell 1 -> ghost 513), timed like the COMB
// bench line: K launches back to back on the same arrays (each launch touches
// > 2 x L2, so every launch also writes back its predecessor's dirty lines).
//
//   row      : one thread per row, both ends (the library's paired x faces)
//   row_pfD  : row + prefetch.global.L2 of the two row ends D rows ahead
//              (rows another CTA will move later: more DRAM requests in flight
//              than the SM's outstanding loads allow)
//   row_z    : row, lanes walk z (32 planes) instead of y
//   row_v2   : two rows per thread (rows r and r + R/2), all four loads first
// Loads after nothing (no PDL here), ld.global.cg; stores plain.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/xface_lab tools/xface_lab.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <algorithm>

constexpr long long N = 514, ROWS = 512LL * 512, NV = 4;
__device__ __forceinline__ long long row_base(long long r) { return (((r / 512) + 1) * N + (r % 512) + 1) * N; }
__device__ __forceinline__ long long row_base_z(long long r) {  // r = y * 512 + z: lanes walk z
    return (((r % 512) + 1) * N + (r / 512) + 1) * N;
}
__device__ __forceinline__ double ldcg(const double* p) {
    double v; asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p)); return v;
}
__device__ __forceinline__ void pf(const void* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }

struct Arr { double* a[NV]; };

template <int MODE, int D>
__global__ void xk(Arr A) {
    const long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (MODE == 3) {  // two rows per thread
        if (t >= NV * ROWS / 2) return;
        const int v = (int)(t / (ROWS / 2));
        const long long r = t % (ROWS / 2);
        double* a = A.a[v];
        const long long b0 = row_base(r), b1 = row_base(r + ROWS / 2);
        const double x0 = ldcg(a + b0 + 1), y0 = ldcg(a + b0 + 512), x1 = ldcg(a + b1 + 1), y1 = ldcg(a + b1 + 512);
        a[b0 + 513] = x0; a[b0] = y0; a[b1 + 513] = x1; a[b1] = y1;
        return;
    }
    if (t >= NV * ROWS) return;
    // MODE 4: consecutive CTAs rotate over the variables (all four progress together)
    const int v = MODE == 4 ? (int)(blockIdx.x % NV) : (int)(t / ROWS);
    const long long r = MODE == 4 ? (long long)(blockIdx.x / NV) * blockDim.x + threadIdx.x : t % ROWS;
    double* a = A.a[v];
    // MODE 5: rows visited in a scattered order (r * 1021 mod ROWS, 1021 prime: a permutation)
    const long long b = MODE == 2 ? row_base_z(r) : (MODE == 5 ? row_base((r * 1021) % ROWS) : row_base(r));
    if (MODE == 1 && r + D < ROWS) {
        const long long bn = row_base(r + D);
        pf(a + bn); pf(a + bn + 512);
    }
    const double x = ldcg(a + b + 1), y = ldcg(a + b + 512);
    a[b + 513] = x;
    a[b] = y;
}

static int g_smem = 0;
template <class F>
static float timeit(F launch, int K) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int i = 0; i < 3; i++) launch();
    std::vector<float> v;
    for (int rep = 0; rep < 5; rep++) {
        cudaEventRecord(e0);
        for (int k = 0; k < K; k++) launch();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        v.push_back(ms * 1e3f / K);
    }
    std::sort(v.begin(), v.end());
    return v[2];
}

int main() {
    Arr A;
    for (int i = 0; i < NV; i++) { cudaMalloc(&A.a[i], N * N * N * 8); cudaMemset(A.a[i], i, N * N * N * 8); }
    const int T = 256, K = 20;
    const long long G = NV * ROWS / T;
    auto pr = [](const char* n, float us) { printf("{\"variant\": \"%s\", \"us_per_launch\": %.2f}\n", n, us); };
    for (int pass = 0; pass < 2; pass++) {
        pr("row", timeit([&] { xk<0, 0><<<G, T>>>(A); }, K));
        pr("row_pf4k", timeit([&] { xk<1, 4096><<<G, T>>>(A); }, K));
        pr("row_pf32k", timeit([&] { xk<1, 32768><<<G, T>>>(A); }, K));
        pr("row_pf128k", timeit([&] { xk<1, 131072><<<G, T>>>(A); }, K));
        pr("row_z", timeit([&] { xk<2, 0><<<G, T>>>(A); }, K));
        pr("row_v2", timeit([&] { xk<3, 0><<<G / 2, T>>>(A); }, K));
        pr("row_varrot", timeit([&] { xk<4, 0><<<G, T>>>(A); }, K));
        pr("row_perm", timeit([&] { xk<5, 0><<<G, T>>>(A); }, K));
        cudaFuncSetAttribute(xk<0, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 110 * 1024);
        cudaFuncSetAttribute(xk<3, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 110 * 1024);
        pr("row_occ4", timeit([&] { xk<0, 0><<<G, T, 50 * 1024>>>(A); }, K));
        pr("row_occ6", timeit([&] { xk<0, 0><<<G, T, 34 * 1024>>>(A); }, K));
        pr("row_v2_occ4", timeit([&] { xk<3, 0><<<G / 2, T, 50 * 1024>>>(A); }, K));
    }
    printf("{\"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
