// netbench.cuh -- microbenchmark of the flush networks (dev instrumentation): one CTA
// of select_kernel's consumer shape sorts P pseudo-random entries to a top-K run,
// `iters` times, and reports the cycles per network call.
#pragma once
#include "cnet.cuh"
#include "network.cuh"
#include "wnet.cuh"

namespace topk {

template <class E>
__device__ __forceinline__ E bench_entry(uint32_t i, uint32_t it);
template <>
__device__ __forceinline__ E32 bench_entry<E32>(uint32_t i, uint32_t it) {
    uint32_t h = (i + 1u) * 0x9E3779B1u ^ (it * 0x85EBCA6Bu);
    h ^= h >> 15;
    h *= 0x2C1B3C6Du;
    h ^= h >> 12;
    return E32::make(h, i);
}
template <>
__device__ __forceinline__ E64 bench_entry<E64>(uint32_t i, uint32_t it) {
    uint32_t h = (i + 1u) * 0x9E3779B1u ^ (it * 0x85EBCA6Bu);
    h ^= h >> 15;
    h *= 0x2C1B3C6Du;
    h ^= h >> 12;
    return E64::make((static_cast<uint64_t>(h) << 32) | h, i);
}

template <class E, int NW>
__global__ void __launch_bounds__(NW * 32, 1) netbench_kernel(int P, int L, int iters, int smem_net,
                                                              unsigned long long* out) {
    extern __shared__ __align__(128) unsigned char smem[];
    SBuf<E> b;
    b.init(smem, 4096);
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned long long total = 0, ta = 0;
    for (int it = 0; it < iters; ++it) {
        for (int i = threadIdx.x; i < P; i += NW * 32) b.st(i, bench_entry<E>(i, it));
        NamedSync<NW * 32>::sync();
        const long long t0 = clock64();
        if (smem_net == 2) {  // barrier cost: 64 named barriers
            for (int q = 0; q < 64; ++q) NamedSync<NW * 32>::sync();
        } else if (smem_net == 3) {  // barrier + one 16-B shared load/store per thread
            for (int q = 0; q < 64; ++q) {
                E x0, x1;
                b.ld2((threadIdx.x * 2 + q * 2) & (P - 1) & ~1, x0, x1);
                NamedSync<NW * 32>::sync();
                b.st2((threadIdx.x * 2 + q * 4) & (P - 1) & ~1, x1, x0);
                NamedSync<NW * 32>::sync();
            }
        } else if (smem_net == 4) {  // code-only network (cnet.cuh) on the P codes
            using C = typename CodeOf<E>::C;
            C* S = reinterpret_cast<C*>(smem + 4096 * 12);
            cnet_topk_codes<E, NW, NamedSync<NW * 32>>(b, P, L < 4 ? 4 : L, S, w, lane);
            if (threadIdx.x == 0 && it == iters - 1) out[2] = static_cast<unsigned long long>(S[0]);
        } else if (smem_net == 5) {  // small-buffer exact network
            if (P <= 512)
                wnet_small<E, 2, NW, NamedSync<NW * 32>>(b, P, L, w, lane);
            else
                wnet_small<E, 4, NW, NamedSync<NW * 32>>(b, P, L, w, lane);
        } else if (smem_net)
            bitonic_topk_smem<E, NW * 32, NamedSync<NW * 32>>(b, P, 1 << L);
        else
            wnet_topk<E, NW, NamedSync<NW * 32>>(b, P, L, w, lane);
        NamedSync<NW * 32>::sync();
        total += static_cast<unsigned long long>(clock64() - t0);
        ta += static_cast<unsigned long long>(g_wnet_phase_a_end - t0);
    }
    if (threadIdx.x == 0) {
        out[0] = total / iters;
        out[1] = ta / iters;
    }
}

}  // namespace topk

namespace topk {

// Debug: the code-only network on n caller-supplied codes (one CTA of the consumer
// shape); writes the top-2^Lp codes best first to out.  Used by the parity tests.
template <class E, int NW>
__global__ void __launch_bounds__(NW * 32, 1) cnet_debug_kernel(
    const typename CodeOf<E>::C* codes, int n, int Lp, typename CodeOf<E>::C* out) {
    using C = typename CodeOf<E>::C;
    extern __shared__ __align__(128) unsigned char smem[];
    SBuf<E> b;
    b.init(smem, 4096);
    C* S = reinterpret_cast<C*>(smem + 4096 * 12);
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < n; i += NW * 32) b.st(i, E::make(codes[i], static_cast<uint32_t>(i)));
    NamedSync<NW * 32>::sync();
    cnet_topk_codes<E, NW, NamedSync<NW * 32>>(b, n, Lp, S, w, lane);
    for (int j = threadIdx.x; j < (1 << Lp); j += NW * 32) out[j] = S[j];
}

}  // namespace topk
