// L2 prefetch-size hint probe for sparse 12-B gathers (configs[2] density).
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <random>
#include <algorithm>
template <int H>
__device__ __forceinline__ unsigned ld4(const unsigned char* p) {
    unsigned v;
    if (H == 0) asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (H == 64) asm volatile("ld.global.nc.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (H == 128) asm volatile("ld.global.nc.L2::128B.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (H == 1) asm volatile("ld.global.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (H == 2) asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (H == 3) asm volatile("ld.global.cs.u32 %0, [%1];" : "=r"(v) : "l"(p));
    else asm volatile("ld.global.nc.L1::no_allocate.L2::256B.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
template <int H>
__global__ void gather12(const unsigned char* __restrict__ src, const long long* __restrict__ off, unsigned char* dst, long long n) {
    long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const unsigned char* p = src + off[i];
    unsigned a = ld4<H>(p), b = ld4<H>(p + 4), c = ld4<H>(p + 8);
    unsigned* d = (unsigned*)(dst + 12 * i);
    d[0] = a; d[1] = b; d[2] = c;
}
int main() {
    long long npoints = 1ll << 26, nseg = npoints / 10;
    std::mt19937_64 rng(20200914);
    std::vector<long long> off(nseg);
    for (long long i = 0; i < nseg; i++) off[i] = (i * 10 + (long long)(rng() % 10)) * 12;
    unsigned char *src, *dst, *fl; long long* doff;
    cudaMalloc(&src, npoints * 12 + 64); cudaMalloc(&dst, nseg * 12); cudaMalloc(&doff, nseg * 8);
    cudaMalloc(&fl, 512 << 20);
    cudaMemcpy(doff, off.data(), nseg * 8, cudaMemcpyHostToDevice);
    cudaMemset(src, 1, npoints * 12);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    long long blocks = (nseg + 255) / 256;
    auto run = [&](int H) {
        float best = 1e9;
        for (int r = 0; r < 7; r++) {
            cudaMemset(fl, r, 512 << 20);
            cudaEventRecord(a);
            switch (H) {
                case 0: gather12<0><<<blocks, 256>>>(src, doff, dst, nseg); break;
                case 64: gather12<64><<<blocks, 256>>>(src, doff, dst, nseg); break;
                case 128: gather12<128><<<blocks, 256>>>(src, doff, dst, nseg); break;
                case 1: gather12<1><<<blocks, 256>>>(src, doff, dst, nseg); break;
                case 2: gather12<2><<<blocks, 256>>>(src, doff, dst, nseg); break;
                case 3: gather12<3><<<blocks, 256>>>(src, doff, dst, nseg); break;
                default: gather12<256><<<blocks, 256>>>(src, doff, dst, nseg); break;
            }
            cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b); best = std::min(best, ms);
        }
        printf("{\"hint\": %d, \"us\": %.1f, \"alg_gbs\": %.1f}\n", H, best * 1e3, 2.0 * nseg * 12 / (best / 1e3) / 1e9);
    };
    for (int H : {0, 64, 128, 256, 1, 2, 3, 0, 64}) run(H);
    return 0;
}
