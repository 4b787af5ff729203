// probe.cuh -- read-bandwidth probes: the paper's "Memory Bandwidth" line, "the time
// taken to read the entire data from global memory ... a lower bound on the runtime of
// any algorithm".  Used by the bench as the measured roofline denominator and
// to choose the streaming mechanism of the top-k pass.
//   * probe_ldg: grid-stride 128-bit non-coherent loads (ld.global.nc.L1::no_allocate),
//     8 in flight per thread, XOR-folded so the loads cannot be dropped.
//   * probe_tma: the exact ring of select_kernel (1 producer warp issuing 1-D bulk
//     copies into `stages` slots of `tile` bytes, 15 consumer warps that wait, read the
//     slot with 128-bit shared loads and release it) -- without the top-k work.
#pragma once
#include "ptx.cuh"

namespace topk {

__device__ __forceinline__ uint4 ld_nc_v4(const uint4* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

__global__ void __launch_bounds__(512) probe_ldg_kernel(const uint4* __restrict__ p, size_t nvec,
                                                        unsigned int* sink) {
    constexpr int U = 8;
    uint32_t acc = 0;
    const size_t stride = static_cast<size_t>(gridDim.x) * blockDim.x;
    size_t i = static_cast<size_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < nvec; i += U * stride) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = ld_nc_v4(p + i + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    for (; i < nvec; i += stride) {
        const uint4 v = ld_nc_v4(p + i);
        acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
    if (acc == 0x9E3779B9u) atomicAdd(sink, 1u);  // practically never; keeps the loads live
}

constexpr int kProbeNC = 480;

__global__ void __launch_bounds__(512, 1) probe_tma_kernel(const unsigned char* __restrict__ p,
                                                          size_t bytes, int tile, int stages,
                                                          unsigned int* sink) {
    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + static_cast<size_t>(stages) * tile);
    uint64_t* empty = full + stages;
    const int tid = threadIdx.x;
    const size_t ntiles = (bytes + tile - 1) / tile;
    const size_t G = gridDim.x, c = blockIdx.x;
    const size_t mine = c < ntiles ? (ntiles - c + G - 1) / G : 0;
    if (tid == 0) {
        for (int s = 0; s < stages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kProbeNC / 32);
        }
        fence_mbar_init();
    }
    __syncthreads();
    if (tid >= kProbeNC) {
        if (tid != kProbeNC) return;
        const uint64_t pol = l2_evict_first_policy();
        for (size_t s = 0; s < mine; ++s) {
            const int slot = static_cast<int>(s % stages);
            if (s >= static_cast<size_t>(stages))
                mbar_wait(&empty[slot], static_cast<uint32_t>((s / stages - 1) & 1));
            const size_t lo = (c + s * G) * tile;
            const uint32_t n = static_cast<uint32_t>(min(static_cast<size_t>(tile), bytes - lo));
            tma_load_1d(smem + static_cast<size_t>(slot) * tile, p + lo, n, &full[slot], pol);
            mbar_arrive_expect_tx(&full[slot], n);
        }
        return;
    }
    uint32_t acc = 0;
    const int nv = tile / 16;
    for (size_t s = 0; s < mine; ++s) {
        const int slot = static_cast<int>(s % stages);
        mbar_wait(&full[slot], static_cast<uint32_t>((s / stages) & 1));
        const uint4* sv = reinterpret_cast<const uint4*>(smem + static_cast<size_t>(slot) * tile);
        for (int j = tid; j < nv; j += kProbeNC) {
            const uint4 v = sv[j];
            acc ^= v.x ^ v.y ^ v.z ^ v.w;
        }
        __syncwarp();
        if ((tid & 31) == 0)
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(&empty[slot]))
                         : "memory");
    }
    if (acc == 0x9E3779B9u) atomicAdd(sink, 1u);
}

}  // namespace topk
