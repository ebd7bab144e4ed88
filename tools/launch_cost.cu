// launch_cost.cu -- diagnostic: host-side cost of the pieces of one small
// ddt_flush on B200 (CUDA 12.9): a kernel launch by parameter size, with and
// without the programmatic-serialisation attribute, and cudaEventRecord.
// Each case: 20000 back-to-back calls, host wall time per call (the GPU side
// is never the bottleneck for these empty kernels).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o launch_cost launch_cost.cu
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <vector>

template <int N> struct P { unsigned char b[N]; };
template <int N> __global__ void k(const __grid_constant__ P<N> p) {
    if (p.b[threadIdx.x % N] == 255 && threadIdx.x == 1000) asm volatile("trap;");
}

template <int N>
static double launch_us(cudaStream_t s, bool pdl, bool ev, cudaEvent_t e) {
    P<N> p{};
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(148);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl ? 1 : 0;
    const int n = 20000;
    for (int i = 0; i < 100; i++) cudaLaunchKernelEx(&cfg, k<N>, p);
    cudaStreamSynchronize(s);
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < n; i++) {
        cudaLaunchKernelEx(&cfg, k<N>, p);
        if (ev) cudaEventRecord(e, s);
    }
    auto t1 = std::chrono::steady_clock::now();
    cudaStreamSynchronize(s);
    return std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
}

int main() {
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEvent_t e;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    for (int rep = 0; rep < 2; rep++) {
        printf("{\"param_B\": 16, \"pdl\": 0, \"event\": 0, \"host_us\": %.3f}\n", launch_us<16>(s, false, false, e));
        printf("{\"param_B\": 16, \"pdl\": 1, \"event\": 0, \"host_us\": %.3f}\n", launch_us<16>(s, true, false, e));
        printf("{\"param_B\": 512, \"pdl\": 1, \"event\": 0, \"host_us\": %.3f}\n", launch_us<512>(s, true, false, e));
        printf("{\"param_B\": 1024, \"pdl\": 1, \"event\": 0, \"host_us\": %.3f}\n", launch_us<1024>(s, true, false, e));
        printf("{\"param_B\": 4096, \"pdl\": 1, \"event\": 0, \"host_us\": %.3f}\n", launch_us<4096>(s, true, false, e));
        printf("{\"param_B\": 4096, \"pdl\": 0, \"event\": 0, \"host_us\": %.3f}\n", launch_us<4096>(s, false, false, e));
        printf("{\"param_B\": 16384, \"pdl\": 1, \"event\": 0, \"host_us\": %.3f}\n", launch_us<16384>(s, true, false, e));
        printf("{\"param_B\": 4096, \"pdl\": 1, \"event\": 1, \"host_us\": %.3f}\n", launch_us<4096>(s, true, true, e));
        printf("{\"param_B\": 16, \"pdl\": 1, \"event\": 1, \"host_us\": %.3f}\n", launch_us<16>(s, true, true, e));
    }
    // other driver calls on the flush path
    const int n = 20000;
    std::vector<cudaEvent_t> evs(n);
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < n; i++) cudaEventCreateWithFlags(&evs[i], cudaEventDisableTiming);
    auto t1 = std::chrono::steady_clock::now();
    printf("{\"call\": \"cudaEventCreateWithFlags\", \"host_us\": %.3f}\n",
           std::chrono::duration<double, std::micro>(t1 - t0).count() / n);
    for (int i = 0; i < n; i++) cudaEventRecord(evs[i], s);
    cudaStreamSynchronize(s);
    t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < n; i++) cudaEventQuery(evs[i]);
    t1 = std::chrono::steady_clock::now();
    printf("{\"call\": \"cudaEventQuery (complete)\", \"host_us\": %.3f}\n",
           std::chrono::duration<double, std::micro>(t1 - t0).count() / n);
    t0 = std::chrono::steady_clock::now();
    int dev = 0;
    for (int i = 0; i < n; i++) cudaGetDevice(&dev);
    t1 = std::chrono::steady_clock::now();
    printf("{\"call\": \"cudaGetDevice\", \"host_us\": %.3f}\n",
           std::chrono::duration<double, std::micro>(t1 - t0).count() / n);
    t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < n; i++) cudaGetLastError();
    t1 = std::chrono::steady_clock::now();
    printf("{\"call\": \"cudaGetLastError\", \"host_us\": %.3f}\n",
           std::chrono::duration<double, std::micro>(t1 - t0).count() / n);
    for (auto e : evs) cudaEventDestroy(e);
    return 0;
}
