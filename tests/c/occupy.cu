// occupy.cu -- TEST SUPPORT ONLY (tests/test_gpu_exchange_protocols.py).
// A kernel that holds SM slots for a bounded time, launched on its own stream
// before a fused exchange: the exchange must still complete (its items are
// claimed by ticket, in item order -- no co-residency assumption).  Thread 0
// of each CTA polls a host-mapped stop word; the others wait at the barrier
// (their slots stay occupied).  Bounded by max_ns so a failing test cannot hang
// the GPU.
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void occupy_kernel(volatile int* stop, volatile unsigned int* started, unsigned long long max_ns) {
    if (threadIdx.x == 0) {
        started[blockIdx.x] = 1u;  // host-mapped, one slot per CTA (no system-scope atomics on host memory)
        __threadfence_system();
        unsigned long long t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        for (;;) {
            if (*stop) break;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > max_ns) break;
            __nanosleep(2000);
        }
    }
    __syncthreads();
}

extern "C" int occupy_launch(void* stream, int ctas, int threads, void* stop, void* started, long long max_ns) {
    // leave the SMs' shared-memory carveout at its maximum: a kernel whose
    // carveout differs from the one an SM runs with cannot be placed on that SM
    // until it drains, whatever its other resources (the exchange kernel needs
    // a little shared memory per CTA)
    cudaFuncSetAttribute(occupy_kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                         (int)cudaSharedmemCarveoutMaxShared);
    occupy_kernel<<<ctas, threads, 0, (cudaStream_t)stream>>>((volatile int*)stop, (volatile unsigned int*)started,
                                                              (unsigned long long)max_ns);
    return (int)cudaGetLastError();
}
