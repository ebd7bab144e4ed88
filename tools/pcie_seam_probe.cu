// pcie_seam_probe.cu -- diagnostic: zero-copy reads of the configs[1] x-face
// cells from a page-locked HOST array (130^3 doubles, rows of 1040 B) into
// device memory, by access pattern:
//   row   : one thread per row reads cell 1 and cell 128 of its row (the paired
//           +x / -x gather the library does), 8-B loads
//   seam  : one thread per row reads cell 128 of row y-1 and cell 1 of row y
//           (the two cells sit in the same 32-B span [y*1040-16, y*1040+16))
//   seam16: as seam, two 16-B loads covering that whole 32-B span
//   one   : one thread per row reads only cell 1 (half the cells: the floor)
// and the matching write patterns into the host array's ghost cells (0, 129).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/pcie_seam_probe tools/pcie_seam_probe.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <algorithm>

constexpr int N = 130;
constexpr int ROWS = 128 * 128;
__device__ __forceinline__ long long rowb(int r) { const int z = 1 + r / 128, y = 1 + r % 128; return ((long long)z * N + y) * N; }

__global__ void rd_row(const double* __restrict__ h, double* o) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < ROWS) { const long long b = rowb(r); o[2 * r] = h[b + 1]; o[2 * r + 1] = h[b + 128]; }
}
__global__ void rd_seam(const double* __restrict__ h, double* o) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < ROWS) { const long long b = rowb(r); o[2 * r] = h[b - 2]; o[2 * r + 1] = h[b + 1]; }
}
__global__ void rd_seam16(const double* __restrict__ h, double* o) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < ROWS) {
        const long long b = rowb(r);
        const double2 lo = *reinterpret_cast<const double2*>(h + b - 2), hi = *reinterpret_cast<const double2*>(h + b);
        o[2 * r] = lo.x; o[2 * r + 1] = hi.y;
    }
}
__global__ void rd_one(const double* __restrict__ h, double* o) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < ROWS) o[r] = h[rowb(r) + 1];
}
__global__ void wr_row(double* h, const double* i) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < ROWS) { const long long b = rowb(r); h[b] = i[2 * r]; h[b + 129] = i[2 * r + 1]; }
}
__global__ void wr_seam(double* h, const double* i) {  // ghost 129 of row y-1 and ghost 0 of row y: adjacent
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r < ROWS) { const long long b = rowb(r); h[b - 1] = i[2 * r]; h[b] = i[2 * r + 1]; }
}

template <class F>
static float t_us(F f) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 3; i++) f();
    std::vector<float> v;
    for (int k = 0; k < 9; k++) {
        cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b); v.push_back(ms * 1e3f);
    }
    std::sort(v.begin(), v.end());
    return v[4];
}

int main() {
    double* h;
    cudaHostAlloc(&h, (size_t)N * N * N * 8, cudaHostAllocMapped);
    for (size_t i = 0; i < (size_t)N * N * N; i++) h[i] = (double)i;
    double* hd;
    cudaHostGetDevicePointer(&hd, h, 0);
    double* o;
    cudaMalloc(&o, 2 * ROWS * 8);
    const int T = 256, G = ROWS / T;
    printf("{\"read_row_us\": %.2f, ", t_us([&] { rd_row<<<G, T>>>(hd, o); }));
    printf("\"read_seam_us\": %.2f, ", t_us([&] { rd_seam<<<G, T>>>(hd, o); }));
    printf("\"read_seam16_us\": %.2f, ", t_us([&] { rd_seam16<<<G, T>>>(hd, o); }));
    printf("\"read_one_us\": %.2f, ", t_us([&] { rd_one<<<G, T>>>(hd, o); }));
    printf("\"write_row_us\": %.2f, ", t_us([&] { wr_row<<<G, T>>>(hd, o); }));
    printf("\"write_seam_us\": %.2f, ", t_us([&] { wr_seam<<<G, T>>>(hd, o); }));
    printf("\"err\": \"%s\"}\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
