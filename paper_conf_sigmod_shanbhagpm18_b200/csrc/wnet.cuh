// wnet.cuh -- register/warp-shuffle form of the paper's operators (K <= 2048; bits >= 9
// of the element index through shared memory).
//
// The paper fuses its operators into kernels whose steps run in shared memory
// ("Operating in Shared Memory") and then combines several steps per thread
// in registers ("Combining/Sequentializing Multiple Steps"; "elements per
// thread B = 16").  On sm_100a the same idea is taken to the warp: a warp holds
// R entries per lane in blocked layout (element e = lane * R + r), so a bitonic step
// on element-index bit b is
//   * b < log2 R : a compare-exchange between two registers of one thread, or
//   * otherwise  : a warp shuffle with lane ^ (1 << (b - log2 R)) -- no shared memory.
// Only the reduction rounds (merge + rebuild of pairs of runs held by different warps)
// go through shared memory, one barrier pair per round.
//
// Step semantics are Alg. 4's generalised to any bit: element e is paired
// with e ^ 2^b; blocks of 2^d elements alternate best-first / worst-first
// (bit d of e == 0 -> best-first); the lower element of a pair in a best-first block
// keeps the better entry.
//
// The step loops are NOT unrolled (only the per-register work is): a fully unrolled
// K = 256 network is ~10^4 distinct instructions per flush and runs out of the
// instruction cache.
#pragma once
#include "keys.cuh"

namespace topk {

template <class E>
__device__ __forceinline__ E shfl_xor_e(const E& e, int m);
template <>
__device__ __forceinline__ E32 shfl_xor_e<E32>(const E32& e, int m) {
    const uint32_t lo = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.v), m);
    const uint32_t hi = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.v >> 32), m);
    return E32{(static_cast<uint64_t>(hi) << 32) | lo};
}
template <>
__device__ __forceinline__ E64 shfl_xor_e<E64>(const E64& e, int m) {
    const uint32_t lo = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.c), m);
    const uint32_t hi = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.c >> 32), m);
    const uint32_t ni = __shfl_xor_sync(0xFFFFFFFFu, e.ni, m);
    return E64{(static_cast<uint64_t>(hi) << 32) | lo, ni};
}

template <>
__device__ __forceinline__ E96 shfl_xor_e<E96>(const E96& e, int m) {
    const uint32_t lo = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.c), m);
    const uint32_t hi = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(e.c >> 32), m);
    const uint32_t c3 = __shfl_xor_sync(0xFFFFFFFFu, e.c3, m);
    const uint32_t ni = __shfl_xor_sync(0xFFFFFFFFu, e.ni, m);
    return E96{(static_cast<uint64_t>(hi) << 32) | lo, c3, ni};
}

// Compare-exchange of two registers: afterwards a holds the better entry iff a_better.
template <class E>
__device__ __forceinline__ void cmpx(E& a, E& b, bool a_better) {
    const bool sw = a_better == better(b, a);  // entries are distinct (or both sentinel)
    const E ta = esel(sw, b, a);
    const E tb = esel(sw, a, b);
    a = ta;
    b = tb;
}

template <int R>
struct Log2 {
    static constexpr int v = 1 + Log2<R / 2>::v;
};
template <>
struct Log2<1> {
    static constexpr int v = 0;
};

// Register step on bit B; wm bit r set <=> register r lies in a worst-first block.
template <class E, int R, int B>
__device__ __forceinline__ void reg_step(E (&x)[R], uint32_t wm) {
#pragma unroll
    for (int r = 0; r < R; ++r)
        if ((r & (1 << B)) == 0) cmpx(x[r], x[r | (1 << B)], ((wm >> r) & 1u) == 0u);
}

// One bitonic step on element bit b with direction bit d (d > b); e0 = element index
// of x[0] of this lane (chunk base + lane * R).
template <class E, int R>
__device__ __forceinline__ void wstep(E (&x)[R], int lane, uint32_t e0, int b, int d) {
    constexpr int LR = Log2<R>::v;
    if (b < LR) {
        // bit r of wm = bit d of register index r (d < LR), or bit d of e0 for all r:
        // the patterns 0xAAAA, 0xCCCC, 0xF0F0, 0xFF00 for d = 0..3 packed in one word
        const uint32_t wm =
            d < LR ? static_cast<uint32_t>((0xFF00F0F0CCCCAAAAull >> (16 * d)) & 0xFFFFull)
                   : (((e0 >> d) & 1u) ? 0xFFFFFFFFu : 0u);
        switch (b) {
            case 0: reg_step<E, R, 0>(x, wm); break;
            case 1: if constexpr (LR > 1) reg_step<E, R, 1>(x, wm); break;
            case 2: if constexpr (LR > 2) reg_step<E, R, 2>(x, wm); break;
            default: if constexpr (LR > 3) reg_step<E, R, 3>(x, wm); break;
        }
    } else {
        const int m = 1 << (b - LR);
        const bool lower = (lane & m) == 0;
        const bool bf = ((e0 >> d) & 1u) == 0u;  // d > b >= LR: same for all r
        const bool keep_better = lower == bf;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const E y = shfl_xor_e(x[r], m);
            x[r] = esel(keep_better == better(y, x[r]), y, x[r]);
        }
    }
}

// Local sort (Alg. 2): runs of length 2^L alternating best-first / worst-first.
template <class E, int R>
__device__ __forceinline__ void wsort_runs(E (&x)[R], int lane, uint32_t e0, int L) {
#pragma unroll 1
    for (int s = 0; s < L; ++s)
#pragma unroll 1
        for (int b = s; b >= 0; --b) wstep<E, R>(x, lane, e0, b, s + 1);
}

// Rebuild (Alg. 4): steps L-1 .. 0 with direction bit L.
template <class E, int R>
__device__ __forceinline__ void wrebuild(E (&x)[R], int lane, uint32_t e0, int L) {
#pragma unroll 1
    for (int b = L - 1; b >= 0; --b) wstep<E, R>(x, lane, e0, b, L);
}

// Entries per lane of a phase-A chunk: 16 (a 512-entry chunk) for 8-byte entries; 8 (256)
// for the 12/16-byte entries of 64-bit codes and compound keys -- 16 of those would take
// 48-64 registers per thread and spill under the kernel's 128-register cap.
#ifndef TOPK_WIDE_R
#define TOPK_WIDE_R 8
#endif
template <class E>
struct WChunk {
    static constexpr int R = sizeof(E) > 8 ? TOPK_WIDE_R : 16;
    static constexpr int B = R == 16 ? 9 : 8;  // element bits inside a chunk
};

// Register pass over 32 R-entry chunks of b[0..P): steps b = hi .. 0 with direction
// bit d (all within a chunk: low bits registers, the next 5 shuffles).
template <class E, int NW>
__device__ __forceinline__ void wchunk_steps(const SBuf<E>& b, int P, int hi, int d, int w,
                                             int lane) {
    constexpr int RA = WChunk<E>::R;
#pragma unroll 1
    for (int base = w * 32 * RA; base < P; base += NW * 32 * RA) {
        E x[RA];
        const int e = base + lane * RA;
#pragma unroll
        for (int r = 0; r < RA; r += 2) {
            if (e + r < P) {
                b.ld2(e + r, x[r], x[r + 1]);
            } else {
                x[r] = E::sentinel();
                x[r + 1] = E::sentinel();
            }
        }
#pragma unroll 1
        for (int bb = hi; bb >= 0; --bb) wstep<E, RA>(x, lane, static_cast<uint32_t>(e), bb, d);
#pragma unroll
        for (int r = 0; r < RA; r += 2)
            if (e + r < P) b.st2(e + r, x[r], x[r + 1]);
    }
}

// Shared-memory step on bit bb >= 9 (pairs in different 512-chunks), Alg. 4 index math.
template <class E, int NT, class Sync>
__device__ __forceinline__ void wsmem_step(const SBuf<E>& b, int P, int bb, int d) {
    const int inc = 1 << bb, dir = 1 << d;
    for (int t = threadIdx.x; t < (P >> 1); t += NT) {
        const int i = (t << 1) - (t & (inc - 1));
        const int j = i + inc;
        const bool best_first = (i & dir) == 0;
        const E x0 = b.ld(i), x1 = b.ld(j);
        const bool sw = best_first == better(x1, x0);
        b.st(i, esel(sw, x1, x0));
        b.st(j, esel(sw, x0, x1));
    }
    Sync::sync();
}

// Bitonic top-K (K = 2^L <= 2048) of b[0..P), P a power of two, 2K <= P <= 4096, by
// the NW warps of the calling group (warp index w, lane), all of which call this.
// Result: b[0..K) best first.  Sync is the group's barrier.  Steps on element bits
// 0-8 run in registers / shuffles; the rare steps on bits 9-10 (K >= 1024) in shared memory.
template <class E, int NW, class Sync>
__device__ void wnet_topk(const SBuf<E>& b, int P, int L, int w, int lane) {
    constexpr int RA = WChunk<E>::R;  // phase A: 32 RA entries per warp chunk
    constexpr int CB = WChunk<E>::B;  // log2 of that
    constexpr int RB = 8;             // phase B: 256 outputs per warp per round
    static_assert(NW * 32 * RB >= 2048, "phase B: one chunk of 256 outputs per warp");
    const int K = 1 << L;
    // Phase A -- local sort into min(K, 2^CB)-runs in registers.  Small buffers use
    // 256-entry chunks (8 per lane) so twice as many warps share the latency-bound
    // step chain; otherwise 32 RA-entry chunks.
    const int LA = L < CB ? L : CB;
    if (L <= 8 && P <= 8 * 256 && NW >= 8) {
        constexpr int R8 = 8;
        const int base = w * 32 * R8;
        if (base < P) {
            E x[R8];
            const int e = base + lane * R8;
#pragma unroll
            for (int r = 0; r < R8; r += 2) {
                if (e + r < P) {
                    b.ld2(e + r, x[r], x[r + 1]);
                } else {
                    x[r] = E::sentinel();
                    x[r + 1] = E::sentinel();
                }
            }
            wsort_runs<E, R8>(x, lane, static_cast<uint32_t>(e), LA);
#pragma unroll
            for (int r = 0; r < R8; r += 2)
                if (e + r < P) b.st2(e + r, x[r], x[r + 1]);
        }
    } else {
#pragma unroll 1
        for (int base = w * 32 * RA; base < P; base += NW * 32 * RA) {
            E x[RA];
            const int e = base + lane * RA;
#pragma unroll
            for (int r = 0; r < RA; r += 2) {
                if (e + r < P) {
                    b.ld2(e + r, x[r], x[r + 1]);
                } else {
                    x[r] = E::sentinel();
                    x[r + 1] = E::sentinel();
                }
            }
            wsort_runs<E, RA>(x, lane, static_cast<uint32_t>(e), LA);
#pragma unroll
            for (int r = 0; r < RA; r += 2)
                if (e + r < P) b.st2(e + r, x[r], x[r + 1]);
        }
    }
    Sync::sync();
    // local-sort stages beyond chunk-size runs: bits >= CB in smem, CB-1 .. 0 in registers
#pragma unroll 1
    for (int d = CB + 1; d <= L; ++d) {
#pragma unroll 1
        for (int bb = d - 1; bb >= CB; --bb) wsmem_step<E, NW * 32, Sync>(b, P, bb, d);
        wchunk_steps<E, NW>(b, P, CB - 1, d, w, lane);
        Sync::sync();
    }
    if (L >= CB) {
        // Phase B for K >= 512: merge through registers + shared memory, rebuild with
        // the same hybrid steps.
#pragma unroll 1
        while (P > K) {
            const int half = P >> 1;
            constexpr int PER = 4096 / 2 / (NW * 32) + 1;
            E keep[PER];
#pragma unroll
            for (int r = 0; r < PER; ++r) {
                const int o = threadIdx.x + r * NW * 32;
                if (o < half) {
                    const int i = (o << 1) - (o & (K - 1));
                    const E a = b.ld(i), c = b.ld(i + K);
                    keep[r] = esel(better(a, c), a, c);
                }
            }
            Sync::sync();
#pragma unroll
            for (int r = 0; r < PER; ++r) {
                const int o = threadIdx.x + r * NW * 32;
                if (o < half) b.st(o, keep[r]);
            }
            Sync::sync();
            P = half;
#pragma unroll 1
            for (int bb = L - 1; bb >= CB; --bb) wsmem_step<E, NW * 32, Sync>(b, P, bb, L);
            wchunk_steps<E, NW>(b, P, CB - 1, L, w, lane);
            Sync::sync();
        }
        return;
    }
    // Phase B -- rounds of merge (keep the better of paired elements of adjacent
    // opposite runs) + rebuild (Alg. 4) until K remain.
#pragma unroll 1
    while (P > K) {
        const int half = P >> 1;
        const int obase = w * 32 * RB;
        const int o0 = obase + lane * RB;
        E x[RB];
        const bool act = obase < half;
        if (act) {
#pragma unroll
            for (int r = 0; r < RB; r += 2) {
                x[r] = E::sentinel();
                x[r + 1] = E::sentinel();
                const int o = o0 + r;
                if (o < half) {
                    if (K == 1) {  // pairs (2o, 2o+1) and (2o+2, 2o+3)
                        E a, c;
                        b.ld2(2 * o, a, c);
                        x[r] = esel(better(a, c), a, c);
                        b.ld2(2 * o + 2, a, c);
                        x[r + 1] = esel(better(a, c), a, c);
                    } else {  // o, o+1 in one run: inputs i, i+1 and i+K, i+K+1
                        const int i = (o << 1) - (o & (K - 1));
                        E a0, a1, c0, c1;
                        b.ld2(i, a0, a1);
                        b.ld2(i + K, c0, c1);
                        x[r] = esel(better(a0, c0), a0, c0);
                        x[r + 1] = esel(better(a1, c1), a1, c1);
                    }
                }
            }
        }
        Sync::sync();
        if (act) {
            wrebuild<E, RB>(x, lane, static_cast<uint32_t>(o0), L);
#pragma unroll
            for (int r = 0; r < RB; r += 2)
                if (o0 + r < half) b.st2(o0 + r, x[r], x[r + 1]);
        }
        Sync::sync();
        P = half;
    }
}

}  // namespace topk

namespace topk {

// Exact bitonic top-K (K = 2^L) of a SMALL buffer b[0..P), 64 <= P <= 1024, P >= 2K --
// the latency form used for the final flushes (a few hundred entries after the
// code-network compaction).  All W = P / (32 R) warps keep R entries per lane for the
// whole network; the paper's rounds of merge + rebuild (Alg. 4) do not compact
// the survivors into fewer warps (that would serialise the rounds on one warp), the
// discarded half just keeps computing.  Element e = w * 32R + lane * R + r: steps on
// bits < log2 R are register compare-exchanges, the next 5 bits warp shuffles, the rest
// exchanges through shared memory -- b[P .. 2P) and b[0 .. P) alternate, so one barrier
// per cross-warp step suffices.  Same step semantics as wstep (Alg. 4 generalised).
template <class E, int R, int B>
__device__ __forceinline__ void wsmall_reg(E (&x)[R], uint32_t e0, int d) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
        if ((r >> B) & 1) continue;
        constexpr int m = 1 << B;
        const bool bf = (((e0 + r) >> d) & 1u) == 0u;
        const E a = x[r], c = x[r | m];
        const bool sw = bf == better(c, a);
        x[r] = esel(sw, c, a);
        x[r | m] = esel(sw, a, c);
    }
}

// One step of wnet_small on element bit bb, blocks best-first iff bit d of e is 0.
template <class E, int R, class Sync>
__device__ __forceinline__ void wsmall_step(E (&x)[R], const SBuf<E>& b, int P, uint32_t e0,
                                            int lane, bool act, int bb, int d, int& region) {
    constexpr int LR = Log2<R>::v;
    if (bb < LR) {
        if (!act) return;
        // compile-time register pairs (a runtime index would put x in local memory)
        if (bb == 0) {
            wsmall_reg<E, R, 0>(x, e0, d);
        } else if (bb == 1) {
            if constexpr (LR > 1) wsmall_reg<E, R, 1>(x, e0, d);
        } else {
            if constexpr (LR > 2) wsmall_reg<E, R, 2>(x, e0, d);
        }
        static_assert(LR <= 3, "wnet_small: at most 8 entries per lane");
    } else if (bb < LR + 5) {
        if (!act) return;
        const int m = 1 << (bb - LR);
        const bool lower = (lane & m) == 0;
        const bool bf = ((e0 >> d) & 1u) == 0u;  // d > bb >= LR: same for every r
        const bool keep_better = lower == bf;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const E y = shfl_xor_e(x[r], m);
            x[r] = esel(keep_better == better(y, x[r]), y, x[r]);
        }
    } else {
        const int base = region * P;
        region ^= 1;
        if (act) {
#pragma unroll
            for (int r = 0; r < R; r += 2) b.st2(base + static_cast<int>(e0) + r, x[r], x[r + 1]);
        }
        Sync::sync();
        if (act) {
            const bool lower = ((e0 >> bb) & 1u) == 0u;
            const bool bf = ((e0 >> d) & 1u) == 0u;
            const bool keep_better = lower == bf;
            const int pe = static_cast<int>(e0 ^ (1u << bb));
#pragma unroll
            for (int r = 0; r < R; r += 2) {
                E y0, y1;
                b.ld2(base + pe + r, y0, y1);
                x[r] = esel(keep_better == better(y0, x[r]), y0, x[r]);
                x[r + 1] = esel(keep_better == better(y1, x[r + 1]), y1, x[r + 1]);
            }
        }
    }
}

// presorted: b already holds runs of 2^L alternating best-first / worst-first (the state
// the local sort leaves) -- only the merge + rebuild rounds run (the merge kernel's
// sorted candidate runs).
template <class E, int R, int NW, class Sync>
__device__ void wnet_small(const SBuf<E>& b, int P, int L, int w, int lane,
                           bool presorted = false) {
    const int W = P / (32 * R);
    const bool act = w < W;
    const uint32_t e0 = static_cast<uint32_t>(w * 32 * R + lane * R);
    int LP = 0;
    while ((1 << LP) < P) ++LP;
    E x[R];
    if (act) {
#pragma unroll
        for (int r = 0; r < R; r += 2) b.ld2(static_cast<int>(e0) + r, x[r], x[r + 1]);
    }
    int region = 1;
#pragma unroll 1
    for (int s = 0; s < (presorted ? 0 : L); ++s)
#pragma unroll 1
        for (int bb = s; bb >= 0; --bb)
            wsmall_step<E, R, Sync>(x, b, P, e0, lane, act, bb, s + 1, region);
#pragma unroll 1
    for (int s = L; s < LP; ++s) {
        // merge: the lower element keeps the better (bit LP of e is 0 everywhere)
        wsmall_step<E, R, Sync>(x, b, P, e0, lane, act, s, LP, region);
#pragma unroll 1
        for (int bb = L - 1; bb >= 0; --bb)
            wsmall_step<E, R, Sync>(x, b, P, e0, lane, act, bb, s + 1, region);
    }
    Sync::sync();  // the last exchange may still be read
    const int K = 1 << L;
    if (act && static_cast<int>(e0) < K) {
#pragma unroll
        for (int r = 0; r < R; r += 2) b.st2(static_cast<int>(e0) + r, x[r], x[r + 1]);
    }
    Sync::sync();
}

}  // namespace topk
