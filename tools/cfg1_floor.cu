// cfg1_floor.cu -- diagnostic: the latency floor of the configs[1] step on
// B200, measured with the most specialised kernel possible (every address a
// compile-time closed form, no descriptors, no work table), timed exactly
// like bench.py times the library: K steps captured in one CUDA graph, each
// step one kernel over the next of R = 96 independent 130^3 double arrays
// (DRAM footprint > 2 x L2), per-step time = graph time / K.
//
// Kernels (the P = 1 self exchange of the 6 faces of a 128^3 interior):
//   empty    : no memory access, 258 CTAs (the graph-node launch floor)
//   faces8   : one thread per 8-B cell (98,304 threads)
//   phased   : z / y face rows as 8-B head + 63 x 16-B + 8-B tail, x-face
//              cells 8 B (66,048 threads; what the library's variant 7 does)
// Prints one JSON line per kernel.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o cfg1_floor cfg1_floor.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

constexpr int N = 130;                       // 128 interior + 2 ghosts
constexpr long long PLANE = (long long)N * N;
__device__ __forceinline__ long long idx(int z, int y, int x) { return ((long long)z * N + y) * N + x; }

__global__ void empty_k(double*) {}
struct Big { unsigned char b[4000]; };
__global__ void empty_big(double*, const __grid_constant__ Big p) { if (p.b[threadIdx.x & 7] == 255 && threadIdx.x == 1000) asm volatile("trap;"); }
// faces8 with a 4-KB parameter block (the size of the library's ParamBatch<8>)
__global__ void faces8_big(double* __restrict__ a, const __grid_constant__ Big p);

// face f: 0: z=1 -> z=129, 1: z=128 -> z=0, 2: y=1 -> y=129, 3: y=128 -> y=0 (r = the other coordinate - 1)
__device__ __forceinline__ void face_rows(int f, int r, long long& s, long long& d) {
    const int o = 1 + r;
    if (f == 0) { s = idx(1, o, 0); d = idx(129, o, 0); }
    else if (f == 1) { s = idx(128, o, 0); d = idx(0, o, 0); }
    else if (f == 2) { s = idx(o, 1, 0); d = idx(o, 129, 0); }
    else { s = idx(o, 128, 0); d = idx(o, 0, 0); }
}

__global__ void faces8(double* __restrict__ a) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t < 4 * 16384) {
        const int f = t / 16384, i = t % 16384, r = i / 128, x = 1 + i % 128;
        long long s, d;
        face_rows(f, r, s, d);
        a[d + x] = __ldg(a + s + x);
    } else if (t < 6 * 16384) {
        const int u = t - 4 * 16384, f = u / 16384, c = u % 16384, z = 1 + c / 128, y = 1 + c % 128;
        if (f == 0) a[idx(z, y, 129)] = __ldg(a + idx(z, y, 1));
        else a[idx(z, y, 0)] = __ldg(a + idx(z, y, 128));
    }
}

__global__ void phased(double* __restrict__ a) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    constexpr int U = 65;  // units per 1024-B row starting at 8 mod 16
    if (t < 4 * 128 * U) {
        const int f = t / (128 * U), r = (t / U) % 128, j = t % U;
        long long s, d;
        face_rows(f, r, s, d);
        const char* ps = reinterpret_cast<const char*>(a + s);
        char* pd = reinterpret_cast<char*>(a + d);
        if (j == 0) *reinterpret_cast<uint2*>(pd + 8) = __ldg(reinterpret_cast<const uint2*>(ps + 8));
        else if (j == U - 1) *reinterpret_cast<uint2*>(pd + 1024) = __ldg(reinterpret_cast<const uint2*>(ps + 1024));
        else *reinterpret_cast<uint4*>(pd + 16 * j) = __ldg(reinterpret_cast<const uint4*>(ps + 16 * j));
    } else if (t < 4 * 128 * U + 2 * 16384) {
        const int u = t - 4 * 128 * U, f = u / 16384, c = u % 16384, z = 1 + c / 128, y = 1 + c % 128;
        if (f == 0) a[idx(z, y, 129)] = __ldg(a + idx(z, y, 1));
        else a[idx(z, y, 0)] = __ldg(a + idx(z, y, 128));
    }
}

__global__ void faces8_big(double* __restrict__ a, const __grid_constant__ Big p) {
    if (p.b[0] == 255 && threadIdx.x == 1000) asm volatile("trap;");
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t < 4 * 16384) {
        const int f = t / 16384, i = t % 16384, r = i / 128, x = 1 + i % 128;
        long long s, d;
        face_rows(f, r, s, d);
        a[d + x] = __ldg(a + s + x);
    } else if (t < 6 * 16384) {
        const int u = t - 4 * 16384, f = u / 16384, c = u % 16384, z = 1 + c / 128, y = 1 + c % 128;
        if (f == 0) a[idx(z, y, 129)] = __ldg(a + idx(z, y, 1));
        else a[idx(z, y, 0)] = __ldg(a + idx(z, y, 128));
    }
}

// ---- PDL variants (what the library does since §7g): trigger on entry,
// address arithmetic, griddepcontrol.wait, then the loads
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__global__ void empty_pdl(double*) { pdl_trigger(); pdl_wait(); }
__global__ void phased_pdl(double* __restrict__ a) {
    pdl_trigger();
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    constexpr int U = 65;
    if (t < 4 * 128 * U) {
        const int f = t / (128 * U), r = (t / U) % 128, j = t % U;
        long long s, d;
        face_rows(f, r, s, d);
        const char* ps = reinterpret_cast<const char*>(a + s);
        char* pd = reinterpret_cast<char*>(a + d);
        pdl_wait();
        if (j == 0) *reinterpret_cast<uint2*>(pd + 8) = __ldg(reinterpret_cast<const uint2*>(ps + 8));
        else if (j == U - 1) *reinterpret_cast<uint2*>(pd + 1024) = __ldg(reinterpret_cast<const uint2*>(ps + 1024));
        else *reinterpret_cast<uint4*>(pd + 16 * j) = __ldg(reinterpret_cast<const uint4*>(ps + 16 * j));
    } else if (t < 4 * 128 * U + 2 * 16384) {
        const int u = t - 4 * 128 * U, f = u / 16384, c = u % 16384, z = 1 + c / 128, y = 1 + c % 128;
        pdl_wait();
        if (f == 0) a[idx(z, y, 129)] = __ldg(a + idx(z, y, 1));
        else a[idx(z, y, 0)] = __ldg(a + idx(z, y, 128));
    } else {
        pdl_wait();
    }
}
// x faces paired: one thread per row moves both of the row's x-face cells
// (x=1 -> x=129 and x=128 -> x=0): the row's two ends are touched together
__global__ void xpair_pdl(double* __restrict__ a) {
    pdl_trigger();
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    constexpr int U = 65;
    if (t < 4 * 128 * U) {
        const int f = t / (128 * U), r = (t / U) % 128, j = t % U;
        long long s, d;
        face_rows(f, r, s, d);
        const char* ps = reinterpret_cast<const char*>(a + s);
        char* pd = reinterpret_cast<char*>(a + d);
        pdl_wait();
        if (j == 0) *reinterpret_cast<uint2*>(pd + 8) = __ldg(reinterpret_cast<const uint2*>(ps + 8));
        else if (j == U - 1) *reinterpret_cast<uint2*>(pd + 1024) = __ldg(reinterpret_cast<const uint2*>(ps + 1024));
        else *reinterpret_cast<uint4*>(pd + 16 * j) = __ldg(reinterpret_cast<const uint4*>(ps + 16 * j));
    } else if (t < 4 * 128 * U + 16384) {
        const int c = t - 4 * 128 * U, z = 1 + c / 128, y = 1 + c % 128;
        pdl_wait();
        const double v1 = __ldg(a + idx(z, y, 1)), v2 = __ldg(a + idx(z, y, 128));
        a[idx(z, y, 129)] = v1;
        a[idx(z, y, 0)] = v2;
    } else {
        pdl_wait();
    }
}
template <class... A>
static void launch_pdl(void (*k)(A...), int grid, cudaStream_t s, A... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k, args...);
}

template <class F>
static double graph_us(F launch, int R, int K) {
    cudaStream_t st;
    cudaStreamCreate(&st);
    for (int k = 0; k < 20; k++) launch(st, k % R);
    cudaStreamSynchronize(st);
    cudaGraph_t g;
    cudaGraphExec_t ge;
    cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
    for (int k = 0; k < K; k++) launch(st, k % R);
    cudaStreamEndCapture(st, &g);
    cudaGraphInstantiate(&ge, g, 0);
    cudaGraphLaunch(ge, st);  // upload
    cudaStreamSynchronize(st);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 5; rep++) {
        cudaEventRecord(e0, st);
        cudaGraphLaunch(ge, st);
        cudaEventRecord(e1, st);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    cudaGraphExecDestroy(ge);
    cudaGraphDestroy(g);
    cudaStreamDestroy(st);
    return best * 1e3 / K;
}

int main() {
    const int R = 96, K = 500;
    double* arr[R];
    for (int r = 0; r < R; r++) {
        cudaMalloc(&arr[r], PLANE * N * sizeof(double));
        cudaMemset(arr[r], r, PLANE * N * sizeof(double));
    }
    const int g8 = (6 * 16384 + 255) / 256, gp = (4 * 128 * 65 + 2 * 16384 + 255) / 256;
    double te = graph_us([&](cudaStream_t s, int r) { empty_k<<<gp, 256, 0, s>>>(arr[r]); }, R, K);
    double t8 = graph_us([&](cudaStream_t s, int r) { faces8<<<g8, 256, 0, s>>>(arr[r]); }, R, K);
    double tp = graph_us([&](cudaStream_t s, int r) { phased<<<gp, 256, 0, s>>>(arr[r]); }, R, K);
    Big big{};
    double teb = graph_us([&](cudaStream_t s, int r) { empty_big<<<gp, 256, 0, s>>>(arr[r], big); }, R, K);
    double t8b = graph_us([&](cudaStream_t s, int r) { faces8_big<<<g8, 256, 0, s>>>(arr[r], big); }, R, K);
    const int gx = (4 * 128 * 65 + 16384 + 255) / 256;
    double tep = graph_us([&](cudaStream_t s, int r) { launch_pdl(empty_pdl, gp, s, arr[r]); }, R, K);
    double tpp = graph_us([&](cudaStream_t s, int r) { launch_pdl(phased_pdl, gp, s, arr[r]); }, R, K);
    double txp = graph_us([&](cudaStream_t s, int r) { launch_pdl(xpair_pdl, gx, s, arr[r]); }, R, K);
    printf("{\"kernel\": \"empty_pdl\", \"ctas\": %d, \"us_per_step\": %.3f}\n", gp, tep);
    printf("{\"kernel\": \"phased_pdl\", \"ctas\": %d, \"us_per_step\": %.3f}\n", gp, tpp);
    printf("{\"kernel\": \"xpair_pdl\", \"ctas\": %d, \"us_per_step\": %.3f}\n", gx, txp);
    printf("{\"kernel\": \"empty\", \"ctas\": %d, \"us_per_step\": %.3f}\n", gp, te);
    printf("{\"kernel\": \"empty_4KB_params\", \"ctas\": %d, \"us_per_step\": %.3f}\n", gp, teb);
    printf("{\"kernel\": \"faces8_4KB_params\", \"ctas\": %d, \"us_per_step\": %.3f}\n", g8, t8b);
    printf("{\"kernel\": \"faces8\", \"ctas\": %d, \"us_per_step\": %.3f}\n", g8, t8);
    printf("{\"kernel\": \"phased\", \"ctas\": %d, \"us_per_step\": %.3f}\n", gp, tp);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
    return 0;
}
