// cnet.cuh -- code-only bitonic top-K: the paper's local sort / merge / rebuild
// (Alg. 4) run on the bare order codes of a CTA's candidate bag.
//
// Why a second network.  The exact network (wnet.cuh) moves (code, index) entries:
// every compare-exchange is a 64-bit compare plus four 32-bit selects, ~7 ALU-pipe
// instructions, and the ALU pipe issues at half rate on sm_100 (B300_MICROARCH.md,
// "rt_SMSP = 2") -- ncu on the exact network shows exactly that bound.  The streaming
// pass mostly needs the network for two things that do not depend on indices:
//   (1) a BOUND: the k-th best code c_k of the bag (>= k entries have code >= c_k, so
//       "code >= c_k" is a valid non-strict bound for the CTA's k-th best entry), and
//       the 2^j-th best codes it publishes for the cross-CTA rank bound;
//   (2) COMPACTION: every entry worse than the bound can be dropped (select.cuh).
// On 32-bit codes a compare-exchange is two VIMNMX (max, min), 3.5x fewer ALU
// instructions; ties and indices are then resolved by the exact network on the few
// survivors only.  Nothing here decides the result -- only which entries can be
// dropped -- so the exactness argument is the bound's.
//
// Layout.  A warp holds a 512-code chunk, 16 codes per lane in blocked order: element
// e = lane * 16 + r (bits 0-3: register r, bits 4-8: lane), as in wnet.cuh.  Steps on
// bits 0-3 are register compare-exchanges, steps on bits 4-8 warp shuffles.
// Direction.  Stage s of the local sort builds runs of 2^(s+1) alternating best-first /
// worst-first by bit D = s+1 of e.  For D <= 3 the direction is a compile-time pattern
// over registers (free: swap the roles of max and min); for D >= 4 it is a per-lane
// bit, handled by storing the codes of worst-first lanes complemented ("transformed
// with D"): every compare-exchange is then "lower element keeps the max", and a stage
// change costs one XOR per code instead of a select per compare-exchange.
#pragma once
#include "keys.cuh"
#include "network.cuh"

namespace topk {

template <class E>
struct CodeOf;
template <>
struct CodeOf<E32> {
    using C = uint32_t;
};
template <>
struct CodeOf<E64> {
    using C = uint64_t;
};
template <>
struct CodeOf<E96> {  // the first 64 bits (keys 1 and 2): a code bound on them is valid
    using C = uint64_t;
};

__device__ __forceinline__ uint32_t ecode(E32 e) { return static_cast<uint32_t>(e.v >> 32); }
__device__ __forceinline__ uint64_t ecode(E64 e) { return e.c; }
__device__ __forceinline__ uint64_t ecode(E96 e) { return e.c; }

__device__ __forceinline__ uint32_t cmax(uint32_t a, uint32_t b) { return max(a, b); }
__device__ __forceinline__ uint32_t cmin(uint32_t a, uint32_t b) { return min(a, b); }
__device__ __forceinline__ uint64_t cmax(uint64_t a, uint64_t b) { return a > b ? a : b; }
__device__ __forceinline__ uint64_t cmin(uint64_t a, uint64_t b) { return a > b ? b : a; }

// up ? min(a, b) : max(a, b) -- two predicated VIMNMX (the compiler would add a SEL).
__device__ __forceinline__ uint32_t cpick(bool up, uint32_t a, uint32_t b) {
    uint32_t r;
    asm("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %3, 0;\n\t"
        "@p min.u32 %0, %1, %2;\n\t@!p max.u32 %0, %1, %2;\n\t}"
        : "=r"(r)
        : "r"(a), "r"(b), "r"(static_cast<uint32_t>(up)));
    return r;
}
__device__ __forceinline__ uint64_t cpick(bool up, uint64_t a, uint64_t b) {
    const bool agt = a > b;
    return (agt != up) ? a : b;
}

__device__ __forceinline__ uint32_t cshfl(uint32_t v, int m) {
    return __shfl_xor_sync(0xFFFFFFFFu, v, m);
}
__device__ __forceinline__ uint64_t cshfl(uint64_t v, int m) {
    const uint32_t lo = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(v), m);
    const uint32_t hi = __shfl_xor_sync(0xFFFFFFFFu, static_cast<uint32_t>(v >> 32), m);
    return (static_cast<uint64_t>(hi) << 32) | lo;
}

template <class C>
__device__ __forceinline__ C lane_mask(int lane, int bit) {
    return ((lane >> bit) & 1) ? ~C(0) : C(0);
}

// Register step on element bit B (< log2 R) with direction bit D:
//   D < 0  : transformed form, lower element keeps the max;
//   D >= 0 : plain form, block best-first iff bit D of the register index is 0.
template <class C, int R, int B, int D>
__device__ __forceinline__ void creg_step(C (&x)[R]) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
        if ((r >> B) & 1) continue;
        const C a = x[r], b = x[r | (1 << B)];
        const C hi = cmax(a, b), lo = cmin(a, b);
        const bool bf = D < 0 ? true : (((r >> (D < 0 ? 0 : D)) & 1) == 0);
        x[r] = bf ? hi : lo;
        x[r | (1 << B)] = bf ? lo : hi;
    }
}

// Register steps B-1 .. 0 in transformed form.
template <class C, int R, int B>
__device__ __forceinline__ void creg_tail(C (&x)[R]) {
    if constexpr (B > 0) {
        creg_step<C, R, B - 1, -1>(x);
        creg_tail<C, R, B - 1>(x);
    }
}

// Shuffle step on lane bit lb: lanes with the bit clear keep the max.
template <class C, int R>
__device__ __forceinline__ void clane_step(C (&x)[R], int lane, int lb) {
    const int m = 1 << lb;
    const bool up = (lane & m) != 0;
#pragma unroll
    for (int r = 0; r < R; ++r) x[r] = cpick(up, x[r], cshfl(x[r], m));
}

// Top-2^L' (L' = Lp in 4..9) codes of one 512-code chunk held in x (blocked layout),
// best first, at elements 0 .. 2^L' - 1 (lanes 0 .. 2^L'/16 - 1) on return.
//   stages 0..L'-1 : local sort into 2^L'-runs (Alg. 2), alternating by bit L';
//   stages L'..8   : merge on bit s (keep the better of each pair) + rebuild
//                    (Alg. 4) of the surviving bitonic runs, direction bit s+1.
template <class C>
__device__ __forceinline__ void cchunk_topk(C (&x)[16], int lane, int Lp) {
    // stages 0-2: 16-register network with compile-time directions (bit D = s+1 of r)
    creg_step<C, 16, 0, 1>(x);
    creg_step<C, 16, 1, 2>(x);
    creg_step<C, 16, 0, 2>(x);
    creg_step<C, 16, 2, 3>(x);
    creg_step<C, 16, 1, 3>(x);
    creg_step<C, 16, 0, 3>(x);
    // stage 3 (D = 4 = lane bit 0): transform, then lower keeps max
    {
        const C m = lane_mask<C>(lane, 0);
#pragma unroll
        for (int r = 0; r < 16; ++r) x[r] ^= m;
    }
    creg_tail<C, 16, 4>(x);
    // stages 4 .. Lp-1: D = s+1 >= 5 (lane bit s-3)
#pragma unroll 1
    for (int s = 4; s < Lp; ++s) {
        const C m = lane_mask<C>(lane, s - 4) ^ lane_mask<C>(lane, s - 3);  // D: s -> s+1
#pragma unroll
        for (int r = 0; r < 16; ++r) x[r] ^= m;
#pragma unroll 1
        for (int b = s; b >= 4; --b) clane_step<C, 16>(x, lane, b - 4);
        creg_tail<C, 16, 4>(x);
    }
    // merge stages: state "transformed with D = s" (lane bit s-4) on entry
#pragma unroll 1
    for (int s = Lp; s < 9; ++s) {
        const int m = 1 << (s - 4);
        // valid data lives in lanes whose bit s-4 is clear (the upper lanes of earlier
        // merges hold discarded entries); the partner lane (bit s-4 set) is complemented
        const C mnext = s + 1 < 9 ? lane_mask<C>(lane, s - 3) : C(0);
#pragma unroll
        for (int r = 0; r < 16; ++r) x[r] = cmax(x[r], ~cshfl(x[r], m)) ^ mnext;
#pragma unroll 1
        for (int b = Lp - 1; b >= 4; --b) clane_step<C, 16>(x, lane, b - 4);
        creg_tail<C, 16, 4>(x);
    }
}

// Rebuild of a bitonic 2^L'-sequence held RB per lane (blocked: element j = lane * RB +
// r within a group of 2^L' / RB lanes), best first.  Steps L'-1 .. 0.
template <class C, int RB>
__device__ __forceinline__ void crebuild(C (&x)[RB], int lane, int Lp) {
    constexpr int LRB = RB == 1 ? 0 : RB == 2 ? 1 : RB == 4 ? 2 : RB == 8 ? 3 : 4;
#pragma unroll 1
    for (int b = Lp - 1; b >= LRB; --b) clane_step<C, RB>(x, lane, b - LRB);
    creg_tail<C, RB, LRB>(x);
}

// One cross-warp round: merge pairs of best-first 2^L'-runs stored at S[(2q << rho) K'],
// S[((2q+1) << rho) K'] (the second read reversed -> a bitonic sequence of pairwise
// maxima) and rebuild; the result replaces the first run.  Warp w takes outputs
// [w * 32 RB, (w+1) * 32 RB).
template <class C, int RB>
__device__ __forceinline__ void cround(C* S, int nout, int Lp, int rho, int w, int lane) {
    const int Kp = 1 << Lp;
    const int o0 = w * 32 * RB + lane * RB;
    if (w * 32 * RB >= nout) return;
    C x[RB];
#pragma unroll
    for (int r = 0; r < RB; ++r) {
        const int o = o0 + r;
        const int q = o >> Lp, j = o & (Kp - 1);
        const C a = S[((2 * q) << rho) * Kp + j];
        const C b = S[((2 * q + 1) << rho) * Kp + (Kp - 1 - j)];
        x[r] = cmax(a, b);
    }
    crebuild<C, RB>(x, lane, Lp);
#pragma unroll
    for (int r = 0; r < RB; ++r) {
        const int o = o0 + r;
        const int q = o >> Lp, j = o & (Kp - 1);
        S[((2 * q) << rho) * Kp + j] = x[r];
    }
}

// Top-K' codes (K' = 2^Lp, 4 <= Lp <= 9) of the entries b[0..n), n <= 512 * NW, best
// first into S[0 .. K').  S must hold nchunks * K' codes (nchunks = P / 512, P =
// max(512, next_pow2(n))).  Positions >= n count as code 0, so S[j] is a valid
// "(j+1)-th best code" only if n > j.  Called by all NW warps of the group (warp w,
// lane); Sync is the group's barrier.  Entry: b consistent; exit: S consistent.
template <class E, int NW, class Sync>
__device__ void cnet_topk_codes(const SBuf<E>& b, int n, int Lp, typename CodeOf<E>::C* S, int w,
                                int lane) {
    using C = typename CodeOf<E>::C;
    int P = 512;
    while (P < n) P <<= 1;
    const int nch = P >> 9;
    const int Kp = 1 << Lp;
    if (w < nch) {
        C x[16];
        const int e0 = w * 512 + lane * 16;
#pragma unroll
        for (int r = 0; r < 16; r += 2) {
            if (e0 + r < n) {
                E p0, p1;
                b.ld2(e0 + r, p0, p1);
                x[r] = ecode(p0);
                x[r + 1] = e0 + r + 1 < n ? ecode(p1) : C(0);
            } else {
                x[r] = C(0);
                x[r + 1] = C(0);
            }
        }
        cchunk_topk<C>(x, lane, Lp);
        // the chunk's top-K' sits at elements e < K' (lanes < K'/16)
        if (lane * 16 < Kp) {
#pragma unroll
            for (int r = 0; r < 16; ++r) S[w * Kp + lane * 16 + r] = x[r];
        }
    }
    Sync::sync();
    int rho = 0;
#pragma unroll 1
    for (int runs = nch; runs > 1; runs >>= 1, ++rho) {
        const int nout = (runs >> 1) * Kp;
        switch (Lp) {
            case 4: cround<C, 1>(S, nout, Lp, rho, w, lane); break;
            case 5: cround<C, 1>(S, nout, Lp, rho, w, lane); break;
            case 6: cround<C, 2>(S, nout, Lp, rho, w, lane); break;
            case 7: cround<C, 4>(S, nout, Lp, rho, w, lane); break;
            case 8: cround<C, 8>(S, nout, Lp, rho, w, lane); break;
            default: cround<C, 16>(S, nout, Lp, rho, w, lane); break;
        }
        Sync::sync();
    }
}

}  // namespace topk

namespace topk {

// Test hook: the code-only network on n caller-supplied codes (one CTA of the consumer
// shape); writes the top-2^Lp codes best first to out (topk_debug_cnet, used by the
// order-statistics parity test).
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
