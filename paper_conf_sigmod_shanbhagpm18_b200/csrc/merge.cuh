// merge.cuh -- the global step of the partitioned top-k: "computing the global top-k
// from the m per-partition heaps" (§1), "the top-k elements emitted by the
// individual core are combined in a final global step" (App. C).  Used after the
// multi-GPU all-gather (§8(e)), after the chunks of an input longer than one launch, and
// after the chunks of a host-resident input.
//
// The candidates arrive as G runs.  When each run is already sorted best first (every
// topk_select result is), the kernel skips the local sort: run 2i is loaded as it is and
// run 2i+1 reversed, so every pair is one bitonic sequence -- exactly the state the
// paper's local sort leaves (Alg. 2: runs alternating direction) -- and log2 G rounds of
// merge (keep the better of paired elements) + rebuild (Alg. 4) leave
// the top-K best first.  Unsorted candidates (topk_merge's general contract) run the
// local sort first.  Inputs with more than one buffer of runs are folded in chunks: the
// running top-K stays in run slot 0 and the next runs fill the other slots.
//
// Entries carry the 64-bit global index as the tie-break (R1) and the row of
// the candidate array for the output gather.  One CTA, entries in registers (R per
// lane) with warp shuffles / shared-memory exchanges (wnet.cuh wnet_small).
#pragma once
#include "keys.cuh"
#include "network.cuh"
#include "wnet.cuh"

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
__device__ __forceinline__ EM shfl_xor_e<EM>(const EM& e, int m) {
    const uint32_t c0 = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.c), m);
    const uint32_t c1 = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.c >> 32), m);
    const uint32_t i0 = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.idx), m);
    const uint32_t i1 = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.idx >> 32), m);
    const uint32_t r = __shfl_xor_sync(0xFFFFFFFFu, e.row, m);
    return EM{(static_cast<uint64_t>(c1) << 32) | c0, (static_cast<uint64_t>(i1) << 32) | i0, r};
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
    __device__ __forceinline__ void ld2(int i, EM& a, EM& b) const {  // i even
        const ulonglong2 q = *reinterpret_cast<const ulonglong2*>(c + i);
        const ulonglong2 x = *reinterpret_cast<const ulonglong2*>(idx + i);
        const uint2 r = *reinterpret_cast<const uint2*>(row + i);
        a = EM{q.x, x.x, r.x};
        b = EM{q.y, x.y, r.y};
    }
    __device__ __forceinline__ void st2(int i, EM a, EM b) const {
        *reinterpret_cast<ulonglong2*>(c + i) = make_ulonglong2(a.c, b.c);
        *reinterpret_cast<ulonglong2*>(idx + i) = make_ulonglong2(a.idx, b.idx);
        *reinterpret_cast<uint2*>(row + i) = make_uint2(a.row, b.row);
    }
};

constexpr int kMergeNT = 512;                     // 16 warps
constexpr int kMergeP = 4096;                     // entries per network buffer
constexpr int kMergeCap = 2 * kMergeP;            // + the exchange region of wnet_small
constexpr size_t kMergeSmem = static_cast<size_t>(kMergeCap) * SBuf<EM>::kBytes;  // 160 KB

struct MergeParams {
    const void* cand_keys;
    const int64_t* cand_idx;
    const uint32_t* cand_payload;
    void* out_keys;
    uint32_t* out_payload;
    int64_t* out_idx;
    uint32_t total;    // candidate entries (runs of run_len, the last one may be shorter)
    uint32_t run_len;  // entries per run
    uint32_t sorted;   // 1: every run is sorted best first (topk_select's output order)
    uint32_t ordered;  // 1 (with sorted): run r's ids all below run r+1's (shards / chunks
                       // in order) -- the position in the candidate array is then as good a
                       // tie-break as the id, and entries narrow to (code, position);
                       // 2: check that on the ids in the kernel (topk_merge_sorted)
    const uint64_t* ranges;  // optional [runs][2] (base, rows) of each run's source: when they
                             // increase run by run the kernel sets `ordered` itself
    uint32_t k, K;
};

// The network over b[0 .. P) (wnet_small: R entries per lane, W = P / (32 R) warps).
template <class Sync>
__device__ __forceinline__ void merge_net(const SBuf<EM>& b, int P, int L, bool presorted, int w,
                                          int lane) {
    if (P <= 1024)
        wnet_small<EM, 2, kMergeNT / 32, Sync>(b, P, L, w, lane, presorted);
    else if (P <= 2048)
        wnet_small<EM, 4, kMergeNT / 32, Sync>(b, P, L, w, lane, presorted);
    else
        wnet_small<EM, 8, kMergeNT / 32, Sync>(b, P, L, w, lane, presorted);
}

// Sorted runs whose ids increase run by run (p.ordered): entries (code, candidate position)
// -- E32 for 32-bit codes (one u64 compare), E64 for f64 -- instead of the 20-byte EM:
// 2-3 words per shuffle instead of 5.  Same rounds as the EM path.
template <class Key, bool MIN, class E>
__device__ __forceinline__ void merge_sorted_narrow(const MergeParams& p, unsigned char* smem,
                                                    int w, int lane) {
    using KT = KeyTraits<Key>;
    SBuf<E> b;
    b.init(smem, kMergeCap);
    const int tid = threadIdx.x;
    const int K = static_cast<int>(p.K), k = static_cast<int>(p.k);
    const int L = __ffs(K) - 1;
    const Key* ck = static_cast<const Key*>(p.cand_keys);
    const uint32_t rl = p.run_len;
    const uint32_t nruns = (p.total + rl - 1) / rl;
    const int use = rl < static_cast<uint32_t>(K) ? static_cast<int>(rl) : K;
    const int slots = kMergeP / K;
    uint32_t next = 0;
    bool first = true;
    while (next < nruns) {
        const int s0 = first ? 0 : 1;
        const uint32_t take = min(static_cast<uint32_t>(slots - s0), nruns - next);
        const int used = s0 + static_cast<int>(take);
        int P = 2 * K;
        while (P < used * K) P <<= 1;
        if (P < 64) P = 64;
        for (int q = tid; q < (P - s0 * K); q += kMergeNT) {
            const int s = s0 + q / K, j = q % K;
            const uint32_t r = next + static_cast<uint32_t>(s - s0);
            E e = E::sentinel();
            if (s < used && j < use) {
                const uint64_t g = static_cast<uint64_t>(r) * rl + j;
                if (g < p.total)
                    e = E::make(KT::template code<MIN>(ck[g]), static_cast<uint32_t>(g));
            }
            b.st(s * K + ((s & 1) ? K - 1 - j : j), e);
        }
        __syncthreads();
        if (P <= 1024)
            wnet_small<E, 2, kMergeNT / 32, CtaSync>(b, P, L, w, lane, true);
        else if (P <= 2048)
            wnet_small<E, 4, kMergeNT / 32, CtaSync>(b, P, L, w, lane, true);
        else
            wnet_small<E, 8, kMergeNT / 32, CtaSync>(b, P, L, w, lane, true);
        next += take;
        first = false;
    }
    for (int j = tid; j < k; j += kMergeNT) {
        const uint32_t row = b.ld(j).lidx();
        if (p.out_idx) p.out_idx[j] = p.cand_idx[row];
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = ck[row];
        if (p.out_payload) p.out_payload[j] = p.cand_payload[row];
    }
}

template <class Key, bool MIN>
__global__ void __launch_bounds__(kMergeNT, 1) merge_kernel(const MergeParams p) {
    using KT = KeyTraits<Key>;
    extern __shared__ __align__(128) unsigned char smem[];
    SBuf<EM> b;
    b.init(smem, kMergeCap);
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int K = static_cast<int>(p.K), k = static_cast<int>(p.k);
    const int L = __ffs(K) - 1;
    const Key* ck = static_cast<const Key*>(p.cand_keys);
    bool ordered = p.sorted && p.ordered == 1u;
    if (p.sorted && p.ordered == 2u && p.total / p.run_len <= kMergeNT) {
        // general sorted runs: check the ids themselves (max of run r < min of run r+1)
        __shared__ unsigned long long s_min[kMergeNT], s_max[kMergeNT];
        __shared__ int s_bad2;
        const uint32_t rl = p.run_len, nr = (p.total + rl - 1) / rl;
        for (uint32_t r = tid; r < nr; r += kMergeNT) {
            s_min[r] = ~0ull;
            s_max[r] = 0ull;
        }
        if (tid == 0) s_bad2 = 0;
        __syncthreads();
        for (uint32_t q = tid; q < p.total; q += kMergeNT) {
            const unsigned long long v = static_cast<unsigned long long>(p.cand_idx[q]);
            atomicMin(&s_min[q / rl], v);
            atomicMax(&s_max[q / rl], v);
        }
        __syncthreads();
        for (uint32_t r = tid; r + 1 < nr; r += kMergeNT)
            if (s_max[r] >= s_min[r + 1]) s_bad2 = 1;
        __syncthreads();
        ordered = s_bad2 == 0;
    }
    if (p.sorted && !ordered && p.ranges) {  // the multi-GPU all-gather: check the shards
        __shared__ int s_bad;
        if (tid == 0) s_bad = 0;
        __syncthreads();
        const uint32_t nr = (p.total + p.run_len - 1) / p.run_len;
        for (uint32_t r = tid; r + 1 < nr; r += kMergeNT)
            if (p.ranges[2 * r] + p.ranges[2 * r + 1] > p.ranges[2 * r + 2]) s_bad = 1;
        __syncthreads();
        ordered = s_bad == 0;
    }
    if (ordered) {
        if constexpr (sizeof(Key) == 4)
            merge_sorted_narrow<Key, MIN, E32>(p, smem, w, lane);
        else
            merge_sorted_narrow<Key, MIN, E64>(p, smem, w, lane);
        return;
    }
    auto entry = [&](uint32_t q) -> EM {
        return EM{static_cast<uint64_t>(KT::template code<MIN>(ck[q])),
                  static_cast<uint64_t>(p.cand_idx[q]), q};
    };
    if (p.sorted) {
        // Runs of min(run_len, K) entries (a sorted run's entries past K never make
        // the top-K); slot 0 holds the running result from the second chunk on.
        const uint32_t rl = p.run_len;
        const uint32_t nruns = (p.total + rl - 1) / rl;
        const int use = rl < static_cast<uint32_t>(K) ? static_cast<int>(rl) : K;
        const int slots = kMergeP / K;  // >= 2 (K <= 2048)
        uint32_t next = 0;
        bool first = true;
        while (next < nruns) {
            const int s0 = first ? 0 : 1;  // slot 0: the result so far (best first)
            const uint32_t take = min(static_cast<uint32_t>(slots - s0), nruns - next);
            const int used = s0 + static_cast<int>(take);
            int P = 2 * K;
            while (P < used * K) P <<= 1;
            if (P < 64) P = 64;
            // load: slot s = run next + s - s0, entries 0 .. use (odd slots reversed)
            for (int q = tid; q < (P - s0 * K); q += kMergeNT) {
                const int s = s0 + q / K, j = q % K;
                const uint32_t r = next + static_cast<uint32_t>(s - s0);
                EM e = EM::sentinel();
                if (s < used && j < use) {
                    const uint64_t g = static_cast<uint64_t>(r) * rl + j;
                    if (g < p.total) e = entry(static_cast<uint32_t>(g));
                }
                b.st(s * K + ((s & 1) ? K - 1 - j : j), e);
            }
            __syncthreads();
            merge_net<CtaSync>(b, P, L, true, w, lane);
            next += take;
            first = false;
        }
    } else {
        // General contract: any order.  Chunks of kMergeP - K new entries next to the
        // running result, local sort + merge + rebuild.
        uint32_t q0 = 0;
        for (bool first = true; q0 < p.total; first = false) {
            const int s0 = first ? 0 : K;
            const int cnt = static_cast<int>(min(static_cast<uint32_t>(kMergeP - s0), p.total - q0));
            int P = 2 * K;
            while (P < s0 + cnt) P <<= 1;
            if (P < 64) P = 64;
            for (int i = tid; i < P - s0; i += kMergeNT)
                b.st(s0 + i, i < cnt ? entry(q0 + static_cast<uint32_t>(i)) : EM::sentinel());
            __syncthreads();
            merge_net<CtaSync>(b, P, L, false, w, lane);
            q0 += static_cast<uint32_t>(cnt);
        }
    }
    for (int j = tid; j < k; j += kMergeNT) {
        const EM e = b.ld(j);
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(e.idx);
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = ck[e.row];
        if (p.out_payload) p.out_payload[j] = p.cand_payload[e.row];
    }
}

}  // namespace topk
