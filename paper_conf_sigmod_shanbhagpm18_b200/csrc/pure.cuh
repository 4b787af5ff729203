// pure.cuh -- TOPK_MODE_PURE for 32-bit keys and K = next_pow2(k) <= 32: the paper's
// data-independent bitonic top-k (every key goes through local sort, merge and rebuild,
// P:143-152; SortReducer P:179-180) as a register/warp-shuffle network, no shared-memory
// bag and no CTA barrier while streaming.
//
// Each warp owns chunks of 1024 keys (32 per lane; key i of the chunk in lane i % 32,
// register i / 32 -- coalesced loads).  Per chunk:
//   (1) keys-only network on the 32-bit order codes (the entries' index is recovered in
//       (3); carrying it through every compare-exchange would triple the work):
//       * local sort (Alg. 2) of each lane's 32 codes into runs of K, in registers;
//       * merge + rebuild (Alg. 4) of those runs inside the lane until one run
//         of K per lane (the halves that lose are dropped: register compaction);
//       * five rounds of merge + rebuild across lanes: the two runs of a lane pair are
//         merged and FOLDED -- each lane of the pair keeps half of the merged bitonic
//         sequence -- so every round halves the registers per lane, as the paper's
//         merge halves the data; once a run lives in one register per lane the losing
//         lanes go idle (sentinel).  The chunk's top-K codes end up sorted best first.
//       Directions: a block that must come out worst first is XOR-complemented, so
//       every compare-exchange is the same max/min pair (the paper's "reverse" flag).
//   (2) tau = the chunk's k-th best code (position k - 1 of that run).
//   (3) exact recovery: the k best entries of the chunk under the full (code, index)
//       order are the codes > tau plus the first (k - #{> tau}) codes == tau in index
//       order (R1) -- ballots over the saved original codes.
//   (4) those k (code, index) entries are sorted (bitonic, one per lane) and merged
//       (merge + rebuild) into the warp's running top-K run.
// At the end the 16 warp runs of a CTA are merged (wnet_small over sorted runs), the CTA
// run goes to the workspace, and the last CTA merges all CTA runs and writes the result.
#pragma once
#include "keys.cuh"
#include "network.cuh"
#include "ptx.cuh"
#include "wnet.cuh"

namespace topk {

constexpr int kPureNT = 512;                       // 16 warps
constexpr int kPureNW = kPureNT / 32;
constexpr int kPureChunk = 1024;                   // keys per warp chunk
constexpr int kPureCap = 4096;                     // merge buffer entries (+ as many for exchange)
constexpr int kPureStages = 3;                     // TMA ring slots per warp (4 KB each)
constexpr int kPureGroup = 16;                     // CTA runs merged per first-level node
// smem: [ring: 16 warps x kPureStages x 4 KB (the merge buffer, 2 x 4096 E32, reuses
// it after streaming) | stage: 16 x 32 E32 | mbarriers: 16 x kPureStages]
constexpr size_t kPureRingBytes = static_cast<size_t>(kPureNW) * kPureStages * kPureChunk * 4;
constexpr size_t kPureSmem = kPureRingBytes + kPureNW * 32 * 8 + kPureNW * kPureStages * 8;
static_assert(kPureRingBytes >= 2 * kPureCap * 8, "merge buffer inside the ring");

struct PureParams {
    const void* keys;
    const uint32_t* payload;
    void* out_keys;
    uint32_t* out_payload;
    int64_t* out_idx;
    unsigned int* ticket;  // workspace words [1 + ceil(G / kPureGroup)], zero on entry and exit
    uint64_t* cand;        // workspace: (G + ceil(G / kPureGroup)) x K E32 (scratch)
    uint64_t n;
    uint64_t base;
    uint32_t k;
    uint32_t L;  // K = 2^L <= 32
};

__device__ __forceinline__ uint32_t pmax(uint32_t a, uint32_t b) { return a > b ? a : b; }
__device__ __forceinline__ uint32_t pmin(uint32_t a, uint32_t b) { return a < b ? a : b; }

// Compare-exchange of registers i < j, best first (larger code to the lower position).
template <int I, int J, int R>
__device__ __forceinline__ void pcx(uint32_t (&x)[R]) {
    const uint32_t hi = pmax(x[I], x[J]), lo = pmin(x[I], x[J]);
    x[I] = hi;
    x[J] = lo;
}

// One in-lane bitonic step on register bit B over x[0 .. N): blocks of 2^D registers
// alternate best first / worst first (D < 32: bit D of the register index; D >= 32:
// every block best first -- a worst-first lane is handled by XOR-complementing).
template <int B, int D, int N, int R>
__device__ __forceinline__ void pstep(uint32_t (&x)[R]) {
#pragma unroll
    for (int r = 0; r < N; ++r) {
        if (r & (1 << B)) continue;
        const int q = r | (1 << B);
        const bool bf = D >= 32 || ((r >> D) & 1) == 0;
        const uint32_t hi = pmax(x[r], x[q]), lo = pmin(x[r], x[q]);
        x[r] = bf ? hi : lo;
        x[q] = bf ? lo : hi;
    }
}

template <int N, int R>
__device__ __forceinline__ void pxor(uint32_t (&x)[R], uint32_t m) {
#pragma unroll
    for (int r = 0; r < N; ++r) x[r] ^= m;
}

// Steps on register bits B .. 0 (descending) with direction bit D.
template <int B, int D, int N, int R>
__device__ __forceinline__ void pdown(uint32_t (&x)[R]) {
    if constexpr (B >= 0) {
        pstep<B, D, N, R>(x);
        pdown<B - 1, D, N, R>(x);
    }
}

// Local sort (Alg. 2) of x[0 .. 32) into runs of 2^L, runs alternating by register bit L;
// stage s (run length 2^(s+1)) uses direction bit s + 1.
template <int S, int L, int R>
__device__ __forceinline__ void plocal(uint32_t (&x)[R]) {
    if constexpr (S < L) {
        pdown<S, S + 1, 32, R>(x);
        plocal<S + 1, L, R>(x);
    }
}

// In-lane merge rounds: runs of K = 2^L in x[0 .. N), N > K: merge pairs (keep the better
// element), compact to N / 2 registers, rebuild (Alg. 4) with direction bit L of
// the new register index -- or, for the last round (N / 2 == K), the lane's direction.
template <int L, int N, int R>
__device__ __forceinline__ void pmerge_in(uint32_t (&x)[R], uint32_t lane_mask) {
    constexpr int K = 1 << L;
    if constexpr (N > K) {
#pragma unroll
        for (int i = 0; i < N / 2; ++i) {
            const int run = i / K, j = i % K;
            x[i] = pmax(x[2 * run * K + j], x[(2 * run + 1) * K + j]);
        }
        if constexpr (N / 2 == K) {
            pxor<K, R>(x, lane_mask);
            pdown<L - 1, 32, K, R>(x);
            pxor<K, R>(x, lane_mask);
        } else {
            pdown<L - 1, L, N / 2, R>(x);
        }
        pmerge_in<L, N / 2, R>(x, lane_mask);
    }
}

// Cross-lane round F (lane pair bit F).  Before it, every run of K spans 2^F lanes with
// Rf = K >> F registers each; run position bits: low log2(Rf) bits = register, the
// others map to lane bits 0 .. F - 1 in reverse (position bit L - 1 - i <-> lane bit i).
// Fold (Rf >= 2): the lower lane keeps merged positions of the low register half, the
// upper lane those of the high half (stored low); then rebuild.  Rf == 1: the upper lane
// goes idle (sentinel 0), the lower keeps the merged element; then rebuild.
template <int F, int L, int R>
__device__ __forceinline__ void pround(uint32_t (&x)[R], int lane) {
    constexpr int K = 1 << L;
    constexpr int Rf = (K >> F) > 1 ? (K >> F) : 1;
    constexpr bool fold = Rf >= 2;
    constexpr int Rn = fold ? Rf / 2 : 1;  // registers per lane after the round
    const bool lower = ((lane >> F) & 1) == 0;
    if constexpr (fold) {
#pragma unroll
        for (int t = 0; t < Rn; ++t) {
            const uint32_t send = lower ? x[t + Rn] : x[t];
            const uint32_t recv = __shfl_xor_sync(0xFFFFFFFFu, send, 1 << F);
            const uint32_t own = lower ? x[t] : x[t + Rn];
            x[t] = pmax(own, recv);
        }
    } else {
        const uint32_t recv = __shfl_xor_sync(0xFFFFFFFFu, x[0], 1 << F);
        x[0] = lower ? pmax(x[0], recv) : 0u;
    }
    // rebuild: blocks best first unless lane bit F + 1 is set (next round's pairing);
    // the last round (F == 4) leaves one best-first run
    const uint32_t m = (F < 4 && ((lane >> (F + 1)) & 1)) ? 0xFFFFFFFFu : 0u;
    pxor<Rn, R>(x, m);
    constexpr int LR = fold ? (L - F - 1) : 0;  // register bits of a position
    // position bits L - 1 .. LR map to lane bits 0 .. L - 1 - LR (reversed), the rest to
    // registers; with Rf == 1 every position bit is a lane bit (runs span 2^L lanes)
#pragma unroll
    for (int pb = L - 1; pb >= LR; --pb) {
        const int lb = L - 1 - pb;
        const bool lo_pos = ((lane >> lb) & 1) == 0;
#pragma unroll
        for (int t = 0; t < Rn; ++t) {
            const uint32_t y = __shfl_xor_sync(0xFFFFFFFFu, x[t], 1 << lb);
            x[t] = lo_pos ? pmax(x[t], y) : pmin(x[t], y);
        }
    }
    if constexpr (LR > 0) pdown<LR - 1, 32, Rn, R>(x);
    pxor<Rn, R>(x, m);
}

template <int F, int L, int R>
__device__ __forceinline__ void prounds(uint32_t (&x)[R], int lane) {
    if constexpr (F < 5) {
        pround<F, L, R>(x, lane);
        prounds<F + 1, L, R>(x, lane);
    }
}

// Lane holding position j of the final run (one register per lane): position bit
// L - 1 - i <-> lane bit i.
__device__ __forceinline__ int pure_pos_lane(int j, int L) {
    return L == 0 ? 0 : static_cast<int>(__brev(static_cast<uint32_t>(j)) >> (32 - L));
}

// Bitonic sort of one E32 per lane over the warp, best first (lane 0 = best).
__device__ __forceinline__ uint64_t warp_sort_e32(uint64_t v, int lane) {
#pragma unroll
    for (int s = 1; s <= 5; ++s) {
#pragma unroll
        for (int b = s - 1; b >= 0; --b) {
            const uint64_t y = __shfl_xor_sync(0xFFFFFFFFu, v, 1 << b);
            const bool bf = s == 5 || ((lane >> s) & 1) == 0;
            const bool lo_pos = ((lane >> b) & 1) == 0;
            v = (lo_pos == bf) ? (v > y ? v : y) : (v < y ? v : y);
        }
    }
    return v;
}


// The warp's chunk loop.  Full chunks arrive by 1-D bulk TMA into the warp's ring
// (kPureStages chunks ahead: the loads overlap the network of earlier chunks); the ragged
// last chunk (and every chunk of a key array that is not 16-byte aligned) is loaded
// directly.
template <class Key, bool MIN, int L>
__device__ __forceinline__ void pure_warp(const PureParams& p, uint32_t* ring, uint64_t* bars,
                                          uint64_t* stage, uint64_t& run, int lane, uint64_t gw,
                                          uint64_t GW) {
    using KT = KeyTraits<Key>;
    constexpr int K = 1 << L;
    const Key* keys = static_cast<const Key*>(p.keys);
    const int k = static_cast<int>(p.k);
    const uint32_t lt = (1u << lane) - 1u;
    const uint64_t nch = (p.n + kPureChunk - 1) / kPureChunk;
    const bool tma = (reinterpret_cast<uintptr_t>(keys) & 15u) == 0;
    const uint64_t nfull = tma ? p.n / kPureChunk : 0;  // chunks that come by TMA
    const int tau_lane = pure_pos_lane(k - 1, L);
    const uint64_t policy = l2_evict_first_policy();
    if (lane == 0) {
        for (int s = 0; s < kPureStages; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
        for (int s = 0; s < kPureStages; ++s) {
            const uint64_t ch = gw + s * GW;
            if (ch < nfull) {
                mbar_arrive_expect_tx(&bars[s], kPureChunk * 4);
                tma_load_1d(ring + s * kPureChunk, keys + ch * kPureChunk, kPureChunk * 4,
                            &bars[s], policy);
            }
        }
    }
    __syncwarp();
    uint32_t it = 0;
#pragma unroll 1
    for (uint64_t ch = gw; ch < nch; ch += GW, ++it) {
        const uint64_t c0 = ch * kPureChunk;
        uint32_t x[32], o[32];
        if (ch < nfull) {
            const int slot = static_cast<int>(it % kPureStages);
            mbar_wait(&bars[slot], (it / kPureStages) & 1u);
            const Key* sk = reinterpret_cast<const Key*>(ring + slot * kPureChunk);
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = KT::template code<MIN>(sk[r * 32 + lane]);
            __syncwarp();
            const uint64_t nx = ch + kPureStages * GW;
            if (lane == 0 && nx < nfull) {
                mbar_arrive_expect_tx(&bars[slot], kPureChunk * 4);
                tma_load_1d(ring + slot * kPureChunk, keys + nx * kPureChunk, kPureChunk * 4,
                            &bars[slot], policy);
            }
        } else {  // ragged last chunk: missing keys are code 0 (never selected below)
#pragma unroll
            for (int r = 0; r < 32; ++r) {
                const uint64_t i = c0 + r * 32 + lane;
                x[r] = i < p.n ? KT::template code<MIN>(keys[i]) : 0u;
            }
        }
#pragma unroll
        for (int r = 0; r < 32; ++r) o[r] = x[r];
        // (1) keys-only network
        const uint32_t lane_mask = (lane & 1) ? 0xFFFFFFFFu : 0u;  // round 0 pairs lanes l, l^1
        if constexpr (L == 5) {
            plocal<0, 4, 32>(x);                 // runs of 16, alternating by register bit 4
            pxor<32, 32>(x, lane_mask);          // last stage: the lane's direction
            pdown<4, 32, 32, 32>(x);
            pxor<32, 32>(x, lane_mask);
        } else if constexpr (L > 0) {
            plocal<0, L, 32>(x);
            pmerge_in<L, 32, 32>(x, lane_mask);
        } else {  // K = 1: max of the lane
#pragma unroll
            for (int r = 1; r < 32; ++r) x[0] = pmax(x[0], x[r]);
        }
        prounds<0, L, 32>(x, lane);
        // (2) tau = k-th best code of the chunk (the run is in lanes 0 .. K - 1)
        const uint32_t tau = __shfl_sync(0xFFFFFFFFu, x[0], tau_lane);
        // run positions before the first code == tau: the codes > tau in the chunk
        const int n_gt = __popc(__ballot_sync(0xFFFFFFFFu, lane < K && x[0] > tau));
        const uint64_t nreal = p.n - c0 < kPureChunk ? p.n - c0 : kPureChunk;
        const int kk = nreal < static_cast<uint64_t>(k) ? static_cast<int>(nreal) : k;
        const int need_eq = kk - n_gt;  // ties at tau, taken in index order (R1)
        // (3) recovery: selected = code > tau, or == tau among the first need_eq ties in
        // index order; key (lane, r) has chunk index r * 32 + lane
        uint32_t gtm = 0u, eqm = 0u;
#pragma unroll
        for (int r = 0; r < 32; ++r) {
            const bool real = nreal == kPureChunk || static_cast<uint64_t>(r * 32 + lane) < nreal;
            gtm |= static_cast<uint32_t>(real && o[r] > tau) << r;
            eqm |= static_cast<uint32_t>(real && o[r] == tau) << r;
        }
        uint32_t selm = gtm | eqm;
        if (__reduce_add_sync(0xFFFFFFFFu, __popc(eqm)) > need_eq) {
            // more ties than needed (tie-heavy input): keep the first need_eq in index
            // order -- register-major, lanes ascending within a register
            selm = gtm;
            int left = need_eq;
#pragma unroll
            for (int r = 0; r < 32; ++r) {
                const uint32_t eq = __ballot_sync(0xFFFFFFFFu, (eqm >> r) & 1u);
                if (((eqm >> r) & 1u) && __popc(eq & lt) < left) selm |= 1u << r;
                left -= __popc(eq);
            }
        }
        // compaction of the kk selected entries (any order: they are sorted below)
        const int cnt = __popc(selm);
        int off = cnt;
#pragma unroll
        for (int o2 = 1; o2 < 32; o2 <<= 1) {
            const int y = __shfl_up_sync(0xFFFFFFFFu, off, o2);
            if (lane >= o2) off += y;
        }
        off -= cnt;
#pragma unroll
        for (int r = 0; r < 32; ++r)
            if ((selm >> r) & 1u)
                stage[off++] = (static_cast<uint64_t>(o[r]) << 32) |
                               static_cast<uint32_t>(~static_cast<uint32_t>(c0 + r * 32 + lane));
        __syncwarp();
        // (4) sort the chunk's k entries and merge them into the running run
        uint64_t v = lane < kk ? stage[lane] : 0ull;
        __syncwarp();
        v = warp_sort_e32(v, lane);
        const uint64_t rev = __shfl_sync(0xFFFFFFFFu, v, (K - 1 - lane) & 31);
        uint64_t m2 = lane < K ? (run > rev ? run : rev) : 0ull;
#pragma unroll
        for (int b = L - 1; b >= 0; --b) {  // rebuild (Alg. 4), best first
            const uint64_t y = __shfl_xor_sync(0xFFFFFFFFu, m2, 1 << b);
            const bool lo_pos = ((lane >> b) & 1) == 0;
            m2 = lo_pos ? (m2 > y ? m2 : y) : (m2 < y ? m2 : y);
        }
        run = m2;
    }
}

// Merge `nruns` sorted (best-first) runs of K entries from global memory (run r at
// src + r * K) into b[0 .. K) best first: slot 0 keeps the result between buffers, odd
// slots are loaded reversed (runs alternating direction: the state the local sort
// leaves), then merge + rebuild rounds (wnet_small, presorted).  Collective (CTA).
template <int L>
__device__ __forceinline__ void merge_runs(const SBuf<E32>& b, const uint64_t* src, int nruns,
                                           int w, int lane) {
    constexpr int K = 1 << L;
    const int tid = threadIdx.x;
    const int slots = kPureCap / K;  // runs per network buffer
    int next = 0;
    bool first = true;
    while (next < nruns) {
        const int s0 = first ? 0 : 1;  // slot 0: the result so far (best first)
        const int take = min(slots - s0, nruns - next);
        const int used = s0 + take;
        int P2 = 2 * K;
        while (P2 < used * K) P2 <<= 1;
        if (P2 < 64) P2 = 64;
        for (int q = tid; q < P2 - s0 * K; q += kPureNT) {
            const int s = s0 + q / K, j = q % K;
            const int r = next + s - s0;
            const E32 e = s < used ? E32{__ldcg(src + static_cast<size_t>(r) * K + j)}
                                   : E32::sentinel();
            b.st(s * K + ((s & 1) ? K - 1 - j : j), e);
        }
        __syncthreads();
        if (P2 <= 1024)
            wnet_small<E32, 2, kPureNW, CtaSync>(b, P2, L, w, lane, true);
        else if (P2 <= 2048)
            wnet_small<E32, 4, kPureNW, CtaSync>(b, P2, L, w, lane, true);
        else
            wnet_small<E32, 8, kPureNW, CtaSync>(b, P2, L, w, lane, true);
        next += take;
        first = false;
    }
}

template <class Key, bool MIN, int L>
__global__ void __launch_bounds__(kPureNT, 1) pure_kernel(const PureParams p) {
    constexpr int K = 1 << L;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ int s_last;
    SBuf<E32> b;
    b.init(smem, 2 * kPureCap);
    uint64_t* stage = reinterpret_cast<uint64_t*>(smem + kPureRingBytes);
    uint64_t* bars = stage + kPureNW * 32;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    // warp chunks interleaved over the CTAs (a small input spreads over every SM)
    const uint64_t gw = static_cast<uint64_t>(w) * gridDim.x + blockIdx.x;
    const uint64_t GW = static_cast<uint64_t>(gridDim.x) * kPureNW;
    uint64_t run = 0ull;  // the warp's running top-K: position = lane (< K), best first
    pure_warp<Key, MIN, L>(p, reinterpret_cast<uint32_t*>(smem) + w * kPureStages * kPureChunk,
                           bars + w * kPureStages, stage + w * 32, run, lane, gw, GW);
    __syncthreads();  // every warp is done with its ring: the merge buffer reuses it
    // CTA: the 16 warp runs, odd ones reversed (sorted runs alternating direction, the
    // state the local sort leaves), merge + rebuild rounds (wnet_small, presorted)
    int P = kPureNW * K;
    if (P < 64) P = 64;
    for (int i = tid; i < P; i += kPureNT) b.st(i, E32::sentinel());
    __syncthreads();
    if (lane < K) b.st(w * K + ((w & 1) ? K - 1 - lane : lane), E32{run});
    __syncthreads();
    wnet_small<E32, 2, kPureNW, CtaSync>(b, P, L, w, lane, true);
    // Reduction tree over the CTA runs, two ticketed levels: the last CTA of each group of
    // kPureGroup merges the group's runs, the last group leader merges the group runs.
    const int G = static_cast<int>(gridDim.x);
    if (G > 1) {
        const int ng = (G + kPureGroup - 1) / kPureGroup;
        const int g = static_cast<int>(blockIdx.x) / kPureGroup;
        const int g0 = g * kPureGroup, gn = min(kPureGroup, G - g0);
        uint64_t* cand = p.cand;                           // G runs
        uint64_t* gcand = p.cand + static_cast<size_t>(G) * K;  // ng group runs
        // (one gpu-scope fence, by the ticket thread after the barrier: cumulative over the
        // run the CTA's threads stored before it; the last CTA's fence after the ticket
        // orders the loads that follow the second barrier)
        for (int j = tid; j < K; j += kPureNT) __stcg(cand + blockIdx.x * K + j, b.ld(j).v);
        __syncthreads();
        if (tid == 0) {
            __threadfence();
            s_last = atomicAdd(p.ticket + 1 + g, 1u) == static_cast<unsigned>(gn - 1);
            if (s_last) __threadfence();
        }
        __syncthreads();
        if (!s_last) return;
        merge_runs<L>(b, cand + static_cast<size_t>(g0) * K, gn, w, lane);
        if (ng > 1) {
            for (int j = tid; j < K; j += kPureNT) __stcg(gcand + g * K + j, b.ld(j).v);
            __syncthreads();
            if (tid == 0) {
                __threadfence();
                s_last = atomicAdd(p.ticket, 1u) == static_cast<unsigned>(ng - 1);
                if (s_last) __threadfence();
            }
            __syncthreads();
            if (!s_last) return;
            merge_runs<L>(b, gcand, ng, w, lane);
        }
        if (tid <= ng) p.ticket[tid] = 0u;  // leave the workspace zeroed (all others done)
    }
    // finalize: best first, original key bits, global index, payload
    const Key* keys = static_cast<const Key*>(p.keys);
    for (int j = tid; j < static_cast<int>(p.k); j += kPureNT) {
        const uint32_t row = b.ld(j).lidx();
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(p.base + row);
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = keys[row];
        if (p.out_payload) p.out_payload[j] = p.payload[row];
    }
}

// ---- K = 64 .. 256: (code, index) entries through the network -------------------------
// A run of K no longer fits the keys-only fold layout with a cheap recovery (K entries of
// every 1024-key chunk would need sorting), so these K carry E32 = code << 32 | ~index
// through every compare-exchange: per 512-key half chunk, 16 entries per lane (position
// lane * 16 + r; key r * 32 + lane of the half, so the shared-memory reads are conflict-
// free), local sort (Alg. 2) into K-runs and merge + rebuild rounds down to one run of K
// (wnet.cuh register / shuffle steps), then merge + rebuild into the warp's running run
// (same layout: positions 0 .. K - 1 in lanes 0 .. K / 16 - 1).

template <class Key, bool MIN, int L>
__device__ __forceinline__ void pure_warp64(const PureParams& p, uint32_t* ring, uint64_t* bars,
                                            E32 (&run)[16], int lane, uint64_t gw, uint64_t GW) {
    using KT = KeyTraits<Key>;
    constexpr int K = 1 << L;
    constexpr int RL = K / 16;  // lanes holding a run
    static_assert(L >= 6 && L <= 8, "pure_warp64: K = 64 .. 256");
    const Key* keys = static_cast<const Key*>(p.keys);
    const uint64_t nch = (p.n + kPureChunk - 1) / kPureChunk;
    const bool tma = (reinterpret_cast<uintptr_t>(keys) & 15u) == 0;
    const uint64_t nfull = tma ? p.n / kPureChunk : 0;
    const uint64_t policy = l2_evict_first_policy();
    const uint32_t e0 = static_cast<uint32_t>(lane * 16);
    if (lane == 0) {
        for (int s = 0; s < kPureStages; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
        for (int s = 0; s < kPureStages; ++s) {
            const uint64_t ch = gw + s * GW;
            if (ch < nfull) {
                mbar_arrive_expect_tx(&bars[s], kPureChunk * 4);
                tma_load_1d(ring + s * kPureChunk, keys + ch * kPureChunk, kPureChunk * 4,
                            &bars[s], policy);
            }
        }
    }
    __syncwarp();
    uint32_t it = 0;
#pragma unroll 1
    for (uint64_t ch = gw; ch < nch; ch += GW, ++it) {
        const uint64_t c0 = ch * kPureChunk;
        const bool full = ch < nfull;
        const int slot = static_cast<int>(it % kPureStages);
        if (full) mbar_wait(&bars[slot], (it / kPureStages) & 1u);
        const Key* sk = reinterpret_cast<const Key*>(ring + slot * kPureChunk);
#pragma unroll 1
        for (int half = 0; half < 2; ++half) {
            E32 x[16];
#pragma unroll
            for (int r = 0; r < 16; ++r) {
                const uint32_t ci = static_cast<uint32_t>(half * 512 + r * 32 + lane);
                const uint64_t i = c0 + ci;
                const Key v = full ? sk[ci] : (i < p.n ? keys[i] : Key{});
                x[r] = i < p.n ? E32::make(KT::template code<MIN>(v), static_cast<uint32_t>(i))
                               : E32::sentinel();
            }
            if (full && half == 1) {  // the slot is consumed: prefetch the chunk after next
                __syncwarp();
                const uint64_t nx = ch + kPureStages * GW;
                if (lane == 0 && nx < nfull) {
                    mbar_arrive_expect_tx(&bars[slot], kPureChunk * 4);
                    tma_load_1d(ring + slot * kPureChunk, keys + nx * kPureChunk, kPureChunk * 4,
                                &bars[slot], policy);
                }
            }
            // local sort (Alg. 2) into K-runs, then merge + rebuild (Alg. 4) rounds
            // to one best-first run of K in positions 0 .. K - 1
            wsort_runs<E32, 16>(x, lane, e0, L);
#pragma unroll 1
            for (int sb = L; sb < 9; ++sb) {
                wstep<E32, 16>(x, lane, e0, sb, 9);  // merge: the lower keeps the better
#pragma unroll 1
                for (int b = L - 1; b >= 0; --b) wstep<E32, 16>(x, lane, e0, b, sb + 1);
            }
            // merge into the running run: run[j] vs chunk[K - 1 - j] (the chunk's run read
            // backwards: lane RL - 1 - l, register 15 - r), then rebuild best first
#pragma unroll
            for (int r = 0; r < 16; ++r) {
                const E32 y = shfl_xor_e(x[15 - r], RL - 1);
                run[r] = lane < RL ? esel(better(run[r], y), run[r], y) : E32::sentinel();
            }
#pragma unroll 1
            for (int b = L - 1; b >= 0; --b) wstep<E32, 16>(run, lane, e0, b, 9);
        }
    }
}

template <class Key, bool MIN, int L>
__global__ void __launch_bounds__(kPureNT, 1) pure64_kernel(const PureParams p) {
    constexpr int K = 1 << L;
    constexpr int RL = K / 16;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ int s_last;
    SBuf<E32> b;
    b.init(smem, 2 * kPureCap);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + kPureRingBytes) + kPureNW * 32;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint64_t gw = static_cast<uint64_t>(w) * gridDim.x + blockIdx.x;
    const uint64_t GW = static_cast<uint64_t>(gridDim.x) * kPureNW;
    E32 run[16];
#pragma unroll
    for (int r = 0; r < 16; ++r) run[r] = E32::sentinel();
    pure_warp64<Key, MIN, L>(p, reinterpret_cast<uint32_t*>(smem) + w * kPureStages * kPureChunk,
                             bars + w * kPureStages, run, lane, gw, GW);
    __syncthreads();  // the merge buffer reuses the rings
    // CTA: the 16 warp runs (odd ones reversed), merge + rebuild rounds (wnet_small)
    if (lane < RL) {
#pragma unroll
        for (int r = 0; r < 16; ++r) {
            const int j = lane * 16 + r;
            b.st(w * K + ((w & 1) ? K - 1 - j : j), run[r]);
        }
    }
    __syncthreads();
    constexpr int P = kPureNW * K;  // 1024 .. 4096
    if constexpr (P <= 1024)
        wnet_small<E32, 2, kPureNW, CtaSync>(b, P, L, w, lane, true);
    else if constexpr (P <= 2048)
        wnet_small<E32, 4, kPureNW, CtaSync>(b, P, L, w, lane, true);
    else
        wnet_small<E32, 8, kPureNW, CtaSync>(b, P, L, w, lane, true);
    const int G = static_cast<int>(gridDim.x);
    if (G > 1) {
        const int ng = (G + kPureGroup - 1) / kPureGroup;
        const int g = static_cast<int>(blockIdx.x) / kPureGroup;
        const int g0 = g * kPureGroup, gn = min(kPureGroup, G - g0);
        uint64_t* cand = p.cand;
        uint64_t* gcand = p.cand + static_cast<size_t>(G) * K;
        // (one gpu-scope fence, by the ticket thread after the barrier: cumulative over the
        // run the CTA's threads stored before it; the last CTA's fence after the ticket
        // orders the loads that follow the second barrier)
        for (int j = tid; j < K; j += kPureNT) __stcg(cand + blockIdx.x * K + j, b.ld(j).v);
        __syncthreads();
        if (tid == 0) {
            __threadfence();
            s_last = atomicAdd(p.ticket + 1 + g, 1u) == static_cast<unsigned>(gn - 1);
            if (s_last) __threadfence();
        }
        __syncthreads();
        if (!s_last) return;
        merge_runs<L>(b, cand + static_cast<size_t>(g0) * K, gn, w, lane);
        if (ng > 1) {
            for (int j = tid; j < K; j += kPureNT) __stcg(gcand + g * K + j, b.ld(j).v);
            __syncthreads();
            if (tid == 0) {
                __threadfence();
                s_last = atomicAdd(p.ticket, 1u) == static_cast<unsigned>(ng - 1);
                if (s_last) __threadfence();
            }
            __syncthreads();
            if (!s_last) return;
            merge_runs<L>(b, gcand, ng, w, lane);
        }
        if (tid <= ng) p.ticket[tid] = 0u;
    }
    const Key* keys = static_cast<const Key*>(p.keys);
    for (int j = tid; j < static_cast<int>(p.k); j += kPureNT) {
        const uint32_t row = b.ld(j).lidx();
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(p.base + row);
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = keys[row];
        if (p.out_payload) p.out_payload[j] = p.payload[row];
    }
}

}  // namespace topk
