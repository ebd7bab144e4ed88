// fused_kernel.cu -- the single fused pack/unpack kernel (sm_100a).
//
// Paper §IV-A.3 (Fig. 6): one kernel executes an array of requests;
// thread blocks are partitioned over requests by size and each runs the device
// function of its request's operation (packing / unpacking), synchronising and
// completing independently.  The paper used Cooperative Groups on V100 to give
// small requests fewer threads.
//
// B200 design: pure HBM-bound byte movement, no tensor
// cores.  The host builds a work table (exclusive prefix sum of per-request
// item counts); every CTA walks items blockIdx.x,
// blockIdx.x + gridDim.x, ... (grid = resident CTAs on 148 SMs), finds its
// request with a binary search of the prefix, caches the descriptor in shared
// memory, and moves kItemVecs vectors of the request's packed stream.  Lane i
// of the CTA takes vectors v0 + i + u*kThreads, so the packed side is perfectly
// coalesced and the strided side is coalesced within each segment.  The vector
// width w (1..16 B) is the largest power of two dividing every segment offset,
// segment length, both user pointers and (count > 1) the extent, so every
// access is naturally aligned; kUnroll independent loads are issued before any
// store (memory-level parallelism).  Vector -> byte offset uses only integer
// arithmetic: 32-bit reciprocal division for the segment index and each
// strided dim (closed form, no metadata), one table lookup for uniform lists,
// one binary search for general lists.  Bytes are moved as integers (uint4,
// uint2, ...): NaN payloads and -0.0 survive bit-exactly.
#include <cuda_runtime.h>
#include <stdint.h>

#include "device_desc.h"

namespace ddt {

__device__ __forceinline__ uint32_t divu(uint32_t n, const DivU32& d) {
    return d.magic ? (uint32_t)__umul64hi((uint64_t)n, d.magic) : n;
}

// Vector width is a runtime, CTA-uniform property of the request (lw = log2 w).
// One code path serves every width: the load / store below is a uniform
// switch around a single instruction, so register allocation does not grow
// with the number of (kind, width) combinations.
template <bool NC>
__device__ __forceinline__ uint4 ld_vec(const uint8_t* p, int lw) {
    uint4 r = make_uint4(0, 0, 0, 0);
    switch (lw) {
    case 4:
        if constexpr (NC)
            asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
        else
            asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
        break;
    case 3:
        if constexpr (NC)
            asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
        else
            asm volatile("ld.global.cg.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
        break;
    case 2:
        if constexpr (NC) asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(r.x) : "l"(p));
        else asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(r.x) : "l"(p));
        break;
    case 1: {
        unsigned short h;
        if constexpr (NC) asm volatile("ld.global.nc.u16 %0, [%1];" : "=h"(h) : "l"(p));
        else asm volatile("ld.global.cg.u16 %0, [%1];" : "=h"(h) : "l"(p));
        r.x = h;
        break;
    }
    default: {
        unsigned short h;
        if constexpr (NC) asm volatile("ld.global.nc.u8 %0, [%1];" : "=h"(h) : "l"(p));
        else asm volatile("ld.global.cg.u8 %0, [%1];" : "=h"(h) : "l"(p));
        r.x = h;
        break;
    }
    }
    return r;
}

__device__ __forceinline__ void st_vec(uint8_t* p, int lw, const uint4& r) {
    switch (lw) {
    case 4: asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w) : "memory"); break;
    case 3: asm volatile("st.global.v2.u32 [%0], {%1,%2};" ::"l"(p), "r"(r.x), "r"(r.y) : "memory"); break;
    case 2: asm volatile("st.global.u32 [%0], %1;" ::"l"(p), "r"(r.x) : "memory"); break;
    case 1: asm volatile("st.global.u16 [%0], %1;" ::"l"(p), "h"((unsigned short)r.x) : "memory"); break;
    default: asm volatile("st.global.u8 [%0], %1;" ::"l"(p), "h"((unsigned short)r.x) : "memory"); break;
    }
}

// Byte offset (relative to the non-contiguous pointer) of vector v.
__device__ __forceinline__ int64_t vec_offset(const ReqDesc& d, uint32_t v) {
    const int lw = d.lw;
    if (d.kind == K_STRIDED) {
        uint32_t s = divu(v, d.vps);
        uint32_t within = v - s * d.vps.d;
        int64_t off = d.base + ((int64_t)within << lw);
        const int nd = d.ndim;
        for (int k = 0; k < nd; k++) {
            uint32_t q = divu(s, d.radix[k]);
            off += (int64_t)(s - q * d.radix[k].d) * d.stride[k];
            s = q;
        }
        return off + (int64_t)s * d.extent;
    } else if (d.kind != K_GENERAL) {
        uint32_t s = divu(v, d.vps);
        uint32_t within = v - s * d.vps.d;
        uint32_t k = divu(s, d.nseg);
        uint32_t j = s - k * d.nseg.d;
        int64_t o = d.kind == K_UNIFORM32 ? (int64_t)__ldg(reinterpret_cast<const int32_t*>(d.list) + j)
                                          : (int64_t)__ldg(reinterpret_cast<const long long*>(d.list) + j);
        return (int64_t)k * d.extent + o + ((int64_t)within << lw);
    } else {
        // general list: instance, then binary search of the packed prefix
        uint32_t k = divu(v, d.vps);
        int64_t pos = (int64_t)(v - k * d.vps.d) << lw;
        const long long* pre = reinterpret_cast<const long long*>(d.prefix);
        uint32_t lo = 0, hi = d.list_n;  // pre[lo] <= pos < pre[hi]
        while (hi - lo > 1) {
            uint32_t mid = (lo + hi) >> 1;
            if (__ldg(pre + mid) <= pos) lo = mid;
            else hi = mid;
        }
        int64_t o = __ldg(reinterpret_cast<const long long*>(d.list) + lo);
        return (int64_t)k * d.extent + o + (pos - __ldg(pre + lo));
    }
}

// COH: the packed side of an unpack is written by another GPU during this
// kernel (P2P exchange) -> read it through L2 (ld.global.cg), never nc/L1.
template <bool COH = false>
__device__ __forceinline__ void run_desc(const ReqDesc& d, uint32_t v0) {
    const uint32_t nvec = d.nvec;
    const int lw = d.lw;
    uint8_t* nc = reinterpret_cast<uint8_t*>(d.noncontig);
    uint8_t* pk = reinterpret_cast<uint8_t*>(d.packed);
    uint4 buf[kUnroll];
    if (d.op == OP_PACK) {
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            uint32_t v = v0 + (uint32_t)(u * kThreads) + threadIdx.x;
            if (v < nvec) buf[u] = ld_vec<true>(nc + vec_offset(d, v), lw);
        }
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            uint32_t v = v0 + (uint32_t)(u * kThreads) + threadIdx.x;
            if (v < nvec) st_vec(pk + ((uint64_t)v << lw), lw, buf[u]);
        }
    } else {
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            uint32_t v = v0 + (uint32_t)(u * kThreads) + threadIdx.x;
            if (v < nvec) buf[u] = ld_vec<!COH>(pk + ((uint64_t)v << lw), lw);
        }
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            uint32_t v = v0 + (uint32_t)(u * kThreads) + threadIdx.x;
            if (v < nvec) st_vec(nc + vec_offset(d, v), lw, buf[u]);
        }
    }
}

// Largest r with prefix[r] <= item (prefix strictly increasing, prefix[0] = 0).
__device__ __forceinline__ uint32_t find_request(const uint32_t* prefix, uint32_t nreq, uint32_t item) {
    uint32_t lo = 0, hi = nreq;
    while (hi - lo > 1) {
        uint32_t mid = (lo + hi) >> 1;
        if (__ldg(prefix + mid) <= item) lo = mid;
        else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(kThreads) ddt_fused_pack_unpack(const uint8_t* __restrict__ table) {
    __shared__ ReqDesc sd;
    const BatchHeader* h = reinterpret_cast<const BatchHeader*>(table);
    const uint32_t nreq = h->nreq;
    const uint32_t total = h->total_items;
    const uint32_t* prefix = reinterpret_cast<const uint32_t*>(table + sizeof(BatchHeader));
    const ReqDesc* descs = reinterpret_cast<const ReqDesc*>(table + h->desc_offset);
    uint32_t cur = 0xffffffffu;
    uint32_t cur_first = 0;
    for (uint32_t item = blockIdx.x; item < total; item += gridDim.x) {
        uint32_t r = find_request(prefix, nreq, item);
        if (r != cur) {
            __syncthreads();
            constexpr int kWords = (int)(sizeof(ReqDesc) / 16);
            if (threadIdx.x < kWords)
                reinterpret_cast<uint4*>(&sd)[threadIdx.x] = __ldg(reinterpret_cast<const uint4*>(descs + r) + threadIdx.x);
            cur_first = __ldg(prefix + r);
            cur = r;
            __syncthreads();
        }
        run_desc(sd, (item - cur_first) * (uint32_t)kItemVecs);
    }
}

// ------------------------------------------------------------------------
// Fused P2P halo exchange: ONE kernel per iteration.
// Pack items store straight into the peer's receive window over NVLink /
// NVSwitch; the CTA completing the last item of a message releases the
// message's epoch flag in the peer's window (the paper's "GPU thread signals
// completion", across GPUs).  Unpack items wait (acquire, system
// scope) on their message's flag and scatter as soon as it arrives -- the
// receiver callback of §IV-B.2 done on the GPU, pack / transfer /
// unpack fused into one launch.  Items are claimed through a global
// ticket and every pack item precedes every unpack item, so pack work never
// waits behind a spinning unpack CTA (deadlock freedom without co-residency).
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void __launch_bounds__(kThreads)
    ddt_fused_exchange(const uint8_t* __restrict__ table, XCtrl* ctrl, int* err_flag, uint64_t timeout_ns) {
    __shared__ ReqDesc sd;
    __shared__ XInfo sx;
    __shared__ uint32_t s_item;
    __shared__ uint64_t s_epoch;
    __shared__ int s_ok;
    const BatchHeader* h = reinterpret_cast<const BatchHeader*>(table);
    const uint32_t nreq = h->nreq;
    const uint32_t total = h->total_items;
    const uint32_t* prefix = reinterpret_cast<const uint32_t*>(table + sizeof(BatchHeader));
    const ReqDesc* descs = reinterpret_cast<const ReqDesc*>(table + h->desc_offset);
    const XInfo* xinfo = reinterpret_cast<const XInfo*>(descs + nreq);
    if (threadIdx.x == 0) s_epoch = *reinterpret_cast<volatile unsigned long long*>(&ctrl->epoch) + 1ull;
    __syncthreads();
    const uint64_t epoch = s_epoch;
    const uint64_t parity = epoch & 1ull;
    uint32_t cur = 0xffffffffu, cur_first = 0;
    for (;;) {
        if (threadIdx.x == 0) s_item = atomicAdd(&ctrl->ticket, 1u);
        __syncthreads();
        const uint32_t item = s_item;
        if (item >= total) break;
        uint32_t r = find_request(prefix, nreq, item);
        if (r != cur) {
            constexpr int kWords = (int)(sizeof(ReqDesc) / 16);
            constexpr int kXWords = (int)(sizeof(XInfo) / 16);
            if (threadIdx.x < kWords)
                reinterpret_cast<uint4*>(&sd)[threadIdx.x] = reinterpret_cast<const uint4*>(descs + r)[threadIdx.x];
            else if (threadIdx.x < kWords + kXWords)
                reinterpret_cast<uint4*>(&sx)[threadIdx.x - kWords] =
                    reinterpret_cast<const uint4*>(xinfo + r)[threadIdx.x - kWords];
            cur_first = prefix[r];
            cur = r;
            __syncthreads();
            if (threadIdx.x == 0) sd.packed += parity * (uint64_t)sx.parity_stride;  // double-buffered window
            __syncthreads();
        }
        const bool is_pack = sd.op == OP_PACK;
        if (!is_pack) {
            if (threadIdx.x == 0) {
                const uint64_t* flag = reinterpret_cast<const uint64_t*>(sx.flag);
                int ok = 1;
                if (ld_acquire_sys(flag) < epoch) {
                    const uint64_t t0 = globaltimer();
                    while (ld_acquire_sys(flag) < epoch) {
                        if (globaltimer() - t0 > timeout_ns) {
                            ok = 0;
                            *reinterpret_cast<volatile int*>(err_flag) = 1;
                            __threadfence_system();
                            break;
                        }
                        __nanosleep(64);
                    }
                }
                s_ok = ok;
            }
            __syncthreads();
            if (s_ok) run_desc<true>(sd, (item - cur_first) * (uint32_t)kItemVecs);
        } else {
            run_desc<false>(sd, (item - cur_first) * (uint32_t)kItemVecs);
            __syncthreads();
            if (threadIdx.x == 0) {
                __threadfence_system();  // this CTA's peer stores before the count (release)
                unsigned long long old = atomicAdd(&ctrl->counters[sx.counter], 1ull);
                if (old + 1ull == epoch * (unsigned long long)sx.nitems) {
                    __threadfence_system();  // acquire the other CTAs' stores, then publish
                    st_release_sys(reinterpret_cast<uint64_t*>(sx.flag), epoch);
                }
            }
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        __threadfence();
        unsigned int n = atomicAdd(&ctrl->done, 1u);
        if (n == gridDim.x - 1) {
            ctrl->ticket = 0;
            ctrl->done = 0;
            *reinterpret_cast<volatile unsigned long long*>(&ctrl->epoch) = epoch;
            __threadfence();
        }
    }
}

static int g_blocks_per_sm = 0;
static int g_xblocks_per_sm = 0;
static int g_sm_count[64];

int device_sm_count(int device) {
    if (device >= 0 && device < 64 && g_sm_count[device] > 0) return g_sm_count[device];
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) n = 148;
    if (device >= 0 && device < 64) g_sm_count[device] = n;
    return n;
}

int launch_exchange(const void* dev_table, uint32_t total_items, void* ctrl, int* err_flag_dev, uint64_t timeout_ns,
                    void* stream, int grid_cap) {
    if (total_items == 0) return 0;
    if (g_xblocks_per_sm == 0) {
        int b = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, ddt_fused_exchange, kThreads, 0) != cudaSuccess || b <= 0)
            b = 4;
        g_xblocks_per_sm = b;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    uint32_t cap = (uint32_t)(device_sm_count(dev) * g_xblocks_per_sm);
    if (grid_cap > 0 && (uint32_t)grid_cap < cap) cap = (uint32_t)grid_cap;
    uint32_t grid = total_items < cap ? total_items : cap;
    ddt_fused_exchange<<<grid, kThreads, 0, (cudaStream_t)stream>>>(reinterpret_cast<const uint8_t*>(dev_table),
                                                                     reinterpret_cast<XCtrl*>(ctrl), err_flag_dev,
                                                                     timeout_ns);
    return (int)cudaGetLastError();
}

int launch_fused(const void* dev_table, uint32_t total_items, void* stream, int grid_cap) {
    if (total_items == 0) return 0;
    if (g_blocks_per_sm == 0) {
        int b = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, ddt_fused_pack_unpack, kThreads, 0) != cudaSuccess || b <= 0)
            b = 4;
        g_blocks_per_sm = b;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    uint32_t cap = (uint32_t)(device_sm_count(dev) * g_blocks_per_sm);
    if (grid_cap > 0 && (uint32_t)grid_cap < cap) cap = (uint32_t)grid_cap;
    uint32_t grid = total_items < cap ? total_items : cap;
    ddt_fused_pack_unpack<<<grid, kThreads, 0, (cudaStream_t)stream>>>(reinterpret_cast<const uint8_t*>(dev_table));
    return (int)cudaGetLastError();
}

}  // namespace ddt

extern "C" int32_t ddt_built_sm(void) { return 100; }
