// merge.cuh -- the global step of the partitioned top-k: "computing the global top-k
// from the m per-partition heaps" (§1), "the top-k elements emitted by the
// individual core are combined in a final global step" (App. C).  Used for the
// multi-GPU path (§8(e)): G ranks' candidate runs -> one exact top-k, with the same
// local sort / merge / rebuild network (network.cuh) over entries that carry a 64-bit
// global index as the tie-break.
#pragma once
#include "keys.cuh"
#include "network.cuh"

namespace topk {

// Entry with a 64-bit global index and the row it came from (for the output gather).
struct EM {
    uint64_t c;
    uint64_t idx;
    uint32_t row;
    __device__ __forceinline__ static EM sentinel() { return EM{0ull, ~0ull, 0u}; }
};
__device__ __forceinline__ bool better(EM a, EM b) {
    return a.c > b.c || (a.c == b.c && a.idx < b.idx);
}
__device__ __forceinline__ EM esel(bool p, EM a, EM b) {
    return EM{sel64(p, a.c, b.c), sel64(p, a.idx, b.idx), sel32(p, a.row, b.row)};
}
template <>
struct SBuf<EM> {
    uint64_t* c;
    uint64_t* idx;
    uint32_t* row;
    static constexpr int kBytes = 20;
    __device__ __forceinline__ void init(unsigned char* base, int cap) {
        c = reinterpret_cast<uint64_t*>(base);
        idx = reinterpret_cast<uint64_t*>(base + 8 * static_cast<size_t>(cap));
        row = reinterpret_cast<uint32_t*>(base + 16 * static_cast<size_t>(cap));
    }
    __device__ __forceinline__ EM ld(int i) const { return EM{c[i], idx[i], row[i]}; }
    __device__ __forceinline__ void st(int i, EM e) const {
        c[i] = e.c;
        idx[i] = e.idx;
        row[i] = e.row;
    }
};

constexpr int kMergeNT = 512;
constexpr int kMergeCap = 8192;
constexpr int kMergeChunk = 4096;
constexpr size_t kMergeSmem = static_cast<size_t>(kMergeCap) * SBuf<EM>::kBytes;

struct MergeParams {
    const void* cand_keys;
    const int64_t* cand_idx;
    const uint32_t* cand_payload;
    void* out_keys;
    uint32_t* out_payload;
    int64_t* out_idx;
    uint32_t total;  // runs * run_len
    uint32_t k, K;
};

template <class Key, bool MIN>
__global__ void __launch_bounds__(kMergeNT, 1) merge_kernel(const MergeParams p) {
    using KT = KeyTraits<Key>;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ int s_cnt;
    SBuf<EM> buf;
    buf.init(smem, kMergeCap);
    const int tid = threadIdx.x, lane = tid & 31;
    const int K = static_cast<int>(p.K), k = static_cast<int>(p.k);
    const int flush_at = kMergeCap - K - kMergeChunk;
    const Key* ck = static_cast<const Key*>(p.cand_keys);
    for (int i = tid; i < K; i += kMergeNT) buf.st(i, EM::sentinel());
    if (tid == 0) s_cnt = 0;
    __syncthreads();

    auto do_flush = [&]() {
        const int cnt = s_cnt;
        int P = K + cnt <= 1 ? 1 : 1 << (32 - __clz(K + cnt - 1));
        if (P < 2 * K) P = 2 * K;
        for (int i = K + cnt + tid; i < P; i += kMergeNT) buf.st(i, EM::sentinel());
        __syncthreads();
        bitonic_topk_smem<EM, kMergeNT, CtaSync>(buf, P, K);
        if (tid == 0) s_cnt = 0;
        __syncthreads();
    };

    constexpr int CI = kMergeChunk / kMergeNT;
    for (uint32_t q0 = 0; q0 < p.total; q0 += kMergeChunk) {
        // Append every candidate of this chunk (warp-aggregated prefix sum).
        int cnt = 0;
        EM ents[CI];
#pragma unroll
        for (int r = 0; r < CI; ++r) {
            const uint32_t q = q0 + tid + r * kMergeNT;
            ents[r] = EM::sentinel();
            if (q < p.total) {
                ents[r] = EM{static_cast<uint64_t>(KT::template code<MIN>(ck[q])),
                             static_cast<uint64_t>(p.cand_idx[q]), q};
                ++cnt;
            }
        }
        int incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
            if (lane >= o) incl += y;
        }
        const int total = __shfl_sync(0xFFFFFFFFu, incl, 31);
        int old = 0;
        if (lane == 31 && total > 0) old = atomicAdd(&s_cnt, total);
        old = __shfl_sync(0xFFFFFFFFu, old, 31);
        int w = K + old + incl - cnt;
#pragma unroll
        for (int r = 0; r < CI; ++r)
            if (q0 + tid + r * kMergeNT < p.total) buf.st(w++, ents[r]);
        const int vote = (lane == 31 && old + total > flush_at) ? 1 : 0;
        if (__syncthreads_or(vote)) do_flush();
    }
    __syncthreads();
    if (s_cnt > 0) do_flush();
    for (int j = tid; j < k; j += kMergeNT) {
        const EM e = buf.ld(j);
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(e.idx);
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = ck[e.row];
        if (p.out_payload) p.out_payload[j] = p.cand_payload[e.row];
    }
}

}  // namespace topk
