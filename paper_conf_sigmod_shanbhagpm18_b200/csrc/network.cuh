// network.cuh -- the paper's three operators on a CTA-resident array of entries.
//
//   local sort  (Alg. 2; pseudocode lost in extraction, reconstructed in
//                SURVEY App. A): runs of length K, alternating best-first / worst-first.
//   merge       (Alg. 3): out[t] = better of the paired elements of adjacent
//                opposite runs -> a bitonic K-sequence holding the pair's top-K; n halves.
//   rebuild     (Alg. 4): re-sort each bitonic K-sequence with the inner loop
//                of the local sort starting at len = K/2.
//
// The compare-exchange index math is Alg. 4's: low = t & (inc-1); i = 2t - low;
// direction from (i & dir) == 0; here "reverse" (Alg. 4 line 7) selects best-first.
// Every compare uses the full entry order (R7: "select the larger element"
// under (code desc, index asc)), so ties are resolved exactly.
//
// This file is the shared-memory form of the network (each step is one pass over
// shared memory separated by barriers -- the paper's "operate in shared memory",
// P:169).  It is used by the flush of the streaming pass and by the merge kernel.
#pragma once
#include "keys.cuh"

namespace topk {

// Barrier over the threads that run the network: the whole CTA, or the 512 consumer
// threads of the streaming pass (named barrier 1; the producer warp never joins).
struct CtaSync {
    __device__ __forceinline__ static void sync() { __syncthreads(); }
};
template <int N>
struct NamedSync {
    __device__ __forceinline__ static void sync() {
        asm volatile("bar.sync 1, %0;" ::"n"(N) : "memory");
    }
};

// One bitonic step over P entries: pairs (i, i + inc); blocks of `dir` entries
// alternate best-first (i & dir == 0) / worst-first.
template <class E, int NT, class Sync>
__device__ __forceinline__ void net_step(const SBuf<E>& b, int P, int inc, int dir) {
    for (int t = threadIdx.x; t < (P >> 1); t += NT) {
        int low = t & (inc - 1);
        int i = (t << 1) - low;
        int j = i + inc;
        bool best_first = (i & dir) == 0;
        const E x0 = b.ld(i), x1 = b.ld(j);
        const bool sw = best_first == better(x1, x0);
        b.st(i, esel(sw, x1, x0));
        b.st(j, esel(sw, x0, x1));
    }
    Sync::sync();
}

// Bitonic top-K of b[0..P) (P, K powers of two, K <= P, P / 2 / NT <= 8).
// On return b[0..K) holds the K best entries, best first.  Requires a barrier-
// consistent buffer on entry; leaves one on exit.
template <class E, int NT, class Sync>
__device__ void bitonic_topk_smem(const SBuf<E>& b, int P, int K) {
    // (1) local sort: sorted runs of length K, alternating direction.
    for (int len = 1; len < K; len <<= 1)
        for (int inc = len; inc > 0; inc >>= 1) net_step<E, NT, Sync>(b, P, inc, len << 1);
    // (2)+(3) merge + rebuild until K remain.
    while (P > K) {
        constexpr int kMaxPer = 8;
        E keep[kMaxPer];
        const int half = P >> 1;
#pragma unroll
        for (int r = 0; r < kMaxPer; ++r) {
            int t = threadIdx.x + r * NT;
            if (t < half) {
                int i = (t << 1) - (t & (K - 1));  // element p of run 2q, partner in run 2q+1
                E a = b.ld(i), c = b.ld(i + K);
                keep[r] = esel(better(a, c), a, c);
            }
        }
        Sync::sync();
#pragma unroll
        for (int r = 0; r < kMaxPer; ++r) {
            int t = threadIdx.x + r * NT;
            if (t < half) b.st(t, keep[r]);
        }
        Sync::sync();
        P = half;
        for (int inc = K >> 1; inc > 0; inc >>= 1) net_step<E, NT, Sync>(b, P, inc, K);
    }
}

}  // namespace topk
