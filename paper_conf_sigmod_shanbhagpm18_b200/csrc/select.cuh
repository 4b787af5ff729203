// select.cuh -- the fused streaming pass: one persistent CTA per SM reads its share of
// the input from HBM exactly once (1-D bulk TMA into a shared-memory ring), keeps the
// keys that can still be in the top-k, and runs the paper's local sort / merge /
// rebuild network over the kept keys together with its running top-K run.  The last
// CTA to finish reduces all CTAs' runs and writes the result (the paper's
// "SortReducer then BitonicReducer until k remain", P:179-180 / P:327, fused into one
// launch: the intermediate candidates live in L2, never in a second HBM pass).
//
// CTA = 16 consumer warps + 1 producer warp.
//   * Producer (one lane): for each of the CTA's tiles -- assigned round-robin through
//     a fixed pseudo-random permutation so that no input order (sorted, reversed) lines
//     up with the scan (the robustness the paper claims for the pure method, P:264/268,
//     is kept by the filter path) -- waits for the ring slot to be empty, issues the
//     bulk copy, and publishes the slot's metadata: tile id and the current threshold
//     (max of the CTA's own k-th best and the global tau_g).
//   * Consumers: per key one compare against the threshold key t (fast test, a superset
//     of "can still be in the top-k"); for the few passing keys the exact entry test
//     and a warp-aggregated append into the survivor buffer (the paper's "buffer
//     filler": prefix sum of matches into a shared-memory buffer).  The buffer
//     is flushed -- bitonic top-K of [running run | survivors | sentinel padding], the
//     paper's local sort + merge + rebuild (network.cuh) -- when it fills; a warp whose
//     survivors do not fit keeps its ring slot, and redoes the tile after the flush.
//   * After each flush the CTA's k-th best is published to tau_g (atomic max): every
//     CTA's k-th best is a valid lower bound of the global k-th best.
#pragma once
#include "keys.cuh"
#include "network.cuh"
#include "ptx.cuh"

namespace topk {

constexpr int kNC = 512;              // consumer threads (16 warps)
constexpr int kNT = kNC + 32;         // + one producer warp
constexpr int kTileBytes = 32768;     // bytes per TMA stage
constexpr int kStages = 4;            // ring depth
constexpr int kCap = 8192;            // survivor buffer entries (incl. the running run)
using CSync = NamedSync<kNC>;

template <class Key>
struct Cfg {
    static constexpr int kTileKeys = kTileBytes / static_cast<int>(sizeof(Key));
    static constexpr int kVecPerThread = kTileBytes / 16 / kNC;
    static constexpr int kItems = kTileKeys / kNC;  // keys per consumer thread per tile
    static_assert(kItems <= 32, "mask width");
};

struct WsHeader {
    unsigned long long tau_g;  // global threshold: max over CTAs of their k-th best
    unsigned int ticket;       // CTAs finished
    unsigned int pad[13];
};
static_assert(sizeof(WsHeader) == 64, "header");

struct SelectParams {
    const void* keys;
    const uint32_t* payload;
    void* out_keys;
    uint32_t* out_payload;
    int64_t* out_idx;
    unsigned char* ws;
    uint64_t n;
    uint64_t base;
    uint64_t body_n;   // keys in the 16-B aligned body (multiple of 16 / sizeof(Key))
    uint32_t head;     // unaligned leading keys (processed as extras by CTA 0)
    uint32_t ntiles;   // tiles of the body
    uint32_t k, K;     // requested k and K = next_pow2(k)
    uint32_t perm_h;   // Feistel half-width (bits); 0 = identity tile order
    uint32_t pad;
};

// Global (workspace) candidate storage, structure of arrays like SBuf.
template <class E>
struct GBuf;
template <>
struct GBuf<E32> {
    uint64_t* v;
    __device__ __forceinline__ void init(unsigned char* base, size_t cap) {
        v = reinterpret_cast<uint64_t*>(base);
        (void)cap;
    }
    __device__ __forceinline__ E32 ld(size_t i) const { return E32{__ldcg(v + i)}; }
    __device__ __forceinline__ void st(size_t i, E32 e) const { __stcg(v + i, e.v); }
};
template <>
struct GBuf<E64> {
    uint64_t* c;
    uint32_t* ni;
    __device__ __forceinline__ void init(unsigned char* base, size_t cap) {
        c = reinterpret_cast<uint64_t*>(base);
        ni = reinterpret_cast<uint32_t*>(base + 8 * cap);
    }
    __device__ __forceinline__ E64 ld(size_t i) const { return E64{__ldcg(c + i), __ldcg(ni + i)}; }
    __device__ __forceinline__ void st(size_t i, E64 e) const {
        __stcg(c + i, e.c);
        __stcg(ni + i, e.ni);
    }
};

// Global threshold publish / read.  E32: the packed entry (exact, with its index).
// E64: the code only, read back as {code, ni = 0} -- i.e. non-strict on that code.
__device__ __forceinline__ void tau_publish(WsHeader* h, E32 e) { atomicMax(&h->tau_g, e.v); }
__device__ __forceinline__ void tau_publish(WsHeader* h, E64 e) { atomicMax(&h->tau_g, e.c); }
template <class E>
__device__ __forceinline__ E tau_from_raw(uint64_t raw);
template <>
__device__ __forceinline__ E32 tau_from_raw<E32>(uint64_t raw) { return E32{raw}; }
template <>
__device__ __forceinline__ E64 tau_from_raw<E64>(uint64_t raw) { return E64{raw, 0u}; }
__device__ __forceinline__ uint64_t tau_load_raw(const WsHeader* h) {
    return ld_relaxed_u64(reinterpret_cast<const uint64_t*>(&h->tau_g));
}

__device__ __forceinline__ E32 load_volatile(const E32* e) {
    return E32{*reinterpret_cast<const volatile uint64_t*>(&e->v)};
}
__device__ __forceinline__ E64 load_volatile(const E64* e) {
    return E64{*reinterpret_cast<const volatile uint64_t*>(&e->c),
               *reinterpret_cast<const volatile uint32_t*>(&e->ni)};
}

// Threshold parameters derived from a bound tau.
template <class E, class Key>
struct Par {
    E tau;
    Key t;                  // a key whose code equals tau's code
    uint32_t strict_after;  // tiles whose first lidx > this may use the strict fast test
    uint32_t active;        // 0 while tau is the sentinel (keep everything)
};

template <class Key, bool MIN>
__device__ __forceinline__ Par<typename KeyTraits<Key>::E, Key> make_par(
    typename KeyTraits<Key>::E tau) {
    Par<typename KeyTraits<Key>::E, Key> p;
    p.tau = tau;
    p.active = tau.is_sentinel() ? 0u : 1u;
    p.t = KeyTraits<Key>::template decode<MIN>(tau.code());
    p.strict_after = tau.lidx();
    return p;
}

// Metadata the producer publishes with each ring slot.
template <class E, class Key>
struct SlotMeta {
    Par<E, Key> par;
    uint32_t tlen;   // keys in this tile
    uint32_t lbase;  // launch-relative row of the tile's first key
};

// Bijection on [0, ntiles): 4-round Feistel on 2h bits with cycle walking.
__device__ __forceinline__ uint32_t tile_of(uint32_t i, uint32_t ntiles, uint32_t h) {
    if (h == 0) return i;
    const uint32_t mask = (1u << h) - 1u;
    uint32_t x = i;
    do {
        uint32_t L = x >> h, R = x & mask;
#pragma unroll
        for (uint32_t r = 0; r < 4; ++r) {
            uint32_t f = R * 0x9E3779B1u + 0x7F4A7C15u * (r + 1u);
            f ^= f >> 15;
            f *= 0x2C1B3C6Du;
            f ^= f >> 12;
            uint32_t nl = R;
            R = L ^ (f & mask);
            L = nl;
        }
        x = (L << h) | R;
    } while (x >= ntiles);
    return x;
}

template <class V>
__device__ __forceinline__ auto vget(const V& v, int w) -> decltype(v.x) {
    if constexpr (sizeof(V) / sizeof(v.x) == 4) {
        return w == 0 ? v.x : w == 1 ? v.y : w == 2 ? v.z : v.w;
    } else {
        return w == 0 ? v.x : v.y;
    }
}

__device__ __forceinline__ int next_pow2_i(int x) {
    return x <= 1 ? 1 : 1 << (32 - __clz(x - 1));
}

// OR-reduction barrier over the consumer warps (named barrier 1).
__device__ __forceinline__ bool cbar_or(bool v) {
    uint32_t r;
    asm volatile(
        "{\n\t.reg .pred p, q;\n\t"
        "setp.ne.u32 p, %1, 0;\n\t"
        "barrier.red.or.pred q, 1, %2, p;\n\t"
        "selp.u32 %0, 1, 0, q;\n\t}"
        : "=r"(r)
        : "r"(static_cast<uint32_t>(v)), "n"(kNC)
        : "memory");
    return r != 0;
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}

// Shared state of one CTA.
template <class E, class Key>
struct CtaState {
    int cnt;          // survivors in buf[K ..)
    int last;         // this CTA reduces all candidates
    uint32_t tau_ver; // seqlock over tau (producer reads it without a barrier)
    E tau;            // CTA bound: its own k-th best, or better
    SlotMeta<E, Key> meta[kStages];
};

// Reserve `total` entries of the survivor buffer (lane 31 of the warp), or fail (-1)
// if they do not fit; the caller then keeps its slot and retries after a flush.
__device__ __forceinline__ int reserve(int* cnt, int total, int limit) {
    int cur = *reinterpret_cast<volatile int*>(cnt);
    while (true) {
        if (cur + total > limit) return -1;
        const int prev = atomicCAS(cnt, cur, cur + total);
        if (prev == cur) return cur;
        cur = prev;
    }
}

// Warp-aggregated append of this thread's kept entries ("computes a prefix sum
// and then writes it out into a shared memory buffer").  Returns the buffer count
// before this warp's entries, or -1 if they did not fit (nothing written).
template <class E, int ITEMS>
__device__ __forceinline__ int append(const SBuf<E>& buf, int* s_cnt, const E (&ents)[ITEMS],
                                      uint32_t mask, int K, int* after) {
    const int lane = threadIdx.x & 31;
    const int cnt = __popc(mask);
    int incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    const int total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    int old = 0;
    if (lane == 31 && total > 0) old = reserve(s_cnt, total, kCap - K);
    old = __shfl_sync(0xFFFFFFFFu, old, 31);
    *after = old + total;
    if (old < 0) return -1;
    int w = K + old + incl - cnt;
#pragma unroll
    for (int q = 0; q < ITEMS; ++q)
        if ((mask >> q) & 1u) buf.st(w++, ents[q]);
    return old;
}

// Collective flush (consumers): bitonic top-K of [run | survivors | padding]; updates
// the CTA bound and publishes it.  Entry: barrier-consistent; exit: same.
template <class Key, bool MIN>
__device__ void flush(const SBuf<typename KeyTraits<Key>::E>& buf,
                      CtaState<typename KeyTraits<Key>::E, Key>* st, WsHeader* hdr, int k,
                      int K) {
    using E = typename KeyTraits<Key>::E;
    const int cnt = st->cnt;
    int P = next_pow2_i(K + cnt);
    if (P < 2 * K) P = 2 * K;
    for (int i = K + cnt + threadIdx.x; i < P; i += kNC) buf.st(i, E::sentinel());
    CSync::sync();
    bitonic_topk_smem<E, kNC, CSync>(buf, P, K);
    if (threadIdx.x == 0) {
        st->cnt = 0;
        const E kth = buf.ld(k - 1);
        if (!kth.is_sentinel()) {
            tau_publish(hdr, kth);
            if (better(kth, st->tau)) {
                volatile uint32_t* ver = &st->tau_ver;
                *ver = *ver + 1u;  // odd: writing
                __threadfence_block();
                st->tau = kth;
                __threadfence_block();
                *ver = *ver + 1u;
            }
        }
    }
    CSync::sync();
}

// Consumer work on one tile held in shared memory: fast test, exact test, append.
// Returns the append result (-1 = did not fit) and sets *vote if a flush is due.
template <class Key, bool MIN, bool FILTER>
__device__ __forceinline__ int consume_tile(const unsigned char* slot_data,
                                            const Par<typename KeyTraits<Key>::E, Key>& pr,
                                            uint32_t tlen, uint32_t lbase,
                                            const SBuf<typename KeyTraits<Key>::E>& buf,
                                            int* s_cnt, int K, int flush_soft, int* vote) {
    using KT = KeyTraits<Key>;
    using E = typename KT::E;
    using Vec = typename KT::Vec;
    using C = Cfg<Key>;
    constexpr int VEC = KT::kVec;
    constexpr int VPT = C::kVecPerThread;
    constexpr int ITEMS = C::kItems;
    constexpr int TK = C::kTileKeys;
    const int tid = threadIdx.x;

    const Vec* sv = reinterpret_cast<const Vec*>(slot_data);
    Vec v[VPT];
#pragma unroll
    for (int j = 0; j < VPT; ++j) v[j] = sv[tid + j * kNC];

    uint32_t mask = 0;
    if (!FILTER || !pr.active) {
        mask = (ITEMS >= 32) ? 0xFFFFFFFFu : ((1u << ITEMS) - 1u);
    } else if (lbase > pr.strict_after) {
#pragma unroll
        for (int q = 0; q < ITEMS; ++q)
            mask |= static_cast<uint32_t>(
                        KT::template fast<MIN, true>(vget(v[q / VEC], q % VEC), pr.t))
                    << q;
    } else {
#pragma unroll
        for (int q = 0; q < ITEMS; ++q)
            mask |= static_cast<uint32_t>(
                        KT::template fast<MIN, false>(vget(v[q / VEC], q % VEC), pr.t))
                    << q;
    }
    if (tlen < static_cast<uint32_t>(TK)) {
#pragma unroll
        for (int q = 0; q < ITEMS; ++q) {
            const uint32_t pos = static_cast<uint32_t>((tid + (q / VEC) * kNC) * VEC + q % VEC);
            if (pos >= tlen) mask &= ~(1u << q);
        }
    }
    *vote = 0;
    if (!__any_sync(0xFFFFFFFFu, mask != 0u)) return 0;
    E ents[ITEMS];
#pragma unroll
    for (int q = 0; q < ITEMS; ++q) {
        ents[q] = E::sentinel();
        if ((mask >> q) & 1u) {
            const uint32_t pos = static_cast<uint32_t>((tid + (q / VEC) * kNC) * VEC + q % VEC);
            const E e = E::make(KT::template code<MIN>(vget(v[q / VEC], q % VEC)), lbase + pos);
            ents[q] = e;
            if (FILTER && pr.active && !better(e, pr.tau)) mask &= ~(1u << q);
        }
    }
    int after = 0;
    const int old = append<E, ITEMS>(buf, s_cnt, ents, mask, K, &after);
    *vote = (old < 0 || after > flush_soft) ? 1 : 0;
    return old;
}

template <class Key, bool MIN, bool FILTER>
__global__ void __launch_bounds__(kNT, 1) select_kernel(const SelectParams p) {
    using KT = KeyTraits<Key>;
    using E = typename KT::E;
    using C = Cfg<Key>;
    constexpr int TK = C::kTileKeys;

    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ CtaState<E, Key> st;

    unsigned char* ring = smem;
    SBuf<E> buf;
    buf.init(smem + static_cast<size_t>(kStages) * kTileBytes, kCap);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + static_cast<size_t>(kStages) * kTileBytes +
                                                 static_cast<size_t>(kCap) * SBuf<E>::kBytes);
    uint64_t* empty = full + kStages;

    const int tid = threadIdx.x;
    const uint32_t G = gridDim.x;
    const uint32_t c = blockIdx.x;
    const int K = static_cast<int>(p.K);
    const int k = static_cast<int>(p.k);
    const int flush_soft = kCap - K - 2048;
    const Key* keys = static_cast<const Key*>(p.keys);
    WsHeader* hdr = reinterpret_cast<WsHeader*>(p.ws);
    const uint32_t my_tiles = c < p.ntiles ? (p.ntiles - c + G - 1) / G : 0u;

    for (int i = tid; i < K; i += kNT) buf.st(i, E::sentinel());
    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kNC / 32);
        }
        fence_mbar_init();
        st.cnt = 0;
        st.tau_ver = 0;
        st.tau = E::sentinel();
    }
    // Extras: the unaligned head and the sub-16-byte tail, appended by CTA 0.
    if (c == 0) {
        const uint64_t tail0 = p.head + p.body_n;
        const int nextra = static_cast<int>(p.head + (p.n - tail0));
        if (tid < nextra) {
            const uint64_t row = tid < static_cast<int>(p.head) ? static_cast<uint64_t>(tid)
                                                                 : tail0 + (tid - p.head);
            buf.st(K + tid, E::make(KT::template code<MIN>(keys[row]), static_cast<uint32_t>(row)));
        }
        if (tid == 0) st.cnt = nextra;
    }
    __syncthreads();

    if (tid >= kNC) {
        // ---------------- producer warp (one lane) ----------------
        if (tid != kNC) return;
        const Key* body = keys + p.head;
        const uint64_t policy = l2_evict_first_policy();
        uint64_t tg_next = FILTER ? tau_load_raw(hdr) : 0ull;
        for (uint32_t s = 0; s < my_tiles; ++s) {
            const int slot = static_cast<int>(s % kStages);
            if (s >= static_cast<uint32_t>(kStages))
                mbar_wait(&empty[slot], ((s / kStages) - 1u) & 1u);
            const uint32_t tile = tile_of(c + s * G, p.ntiles, p.perm_h);
            const uint64_t lo = static_cast<uint64_t>(tile) * TK;
            const uint64_t len = min(static_cast<uint64_t>(TK), p.body_n - lo);
            const uint32_t bytes = static_cast<uint32_t>(len * sizeof(Key));
            tma_load_1d(ring + static_cast<size_t>(slot) * kTileBytes, body + lo, bytes,
                        &full[slot], policy);
            SlotMeta<E, Key> m;
            m.tlen = static_cast<uint32_t>(len);
            m.lbase = static_cast<uint32_t>(p.head + lo);
            if (FILTER) {
                const E tg = tau_from_raw<E>(tg_next);
                tg_next = tau_load_raw(hdr);  // prefetch for the next tile
                E tl;
                uint32_t v1, v2;
                do {
                    v1 = *reinterpret_cast<volatile uint32_t*>(&st.tau_ver);
                    __threadfence_block();
                    tl = load_volatile(&st.tau);
                    __threadfence_block();
                    v2 = *reinterpret_cast<volatile uint32_t*>(&st.tau_ver);
                } while (v1 != v2 || (v1 & 1u));
                m.par = make_par<Key, MIN>(better(tg, tl) ? tg : tl);
            } else {
                m.par = make_par<Key, MIN>(E::sentinel());
            }
            st.meta[slot] = m;
            mbar_arrive_expect_tx(&full[slot], bytes);  // release: meta visible with data
        }
        return;
    }

    // ---------------- consumer warps ----------------
    const int lane = tid & 31;
    for (uint32_t s = 0; s < my_tiles; ++s) {
        const int slot = static_cast<int>(s % kStages);
        mbar_wait(&full[slot], (s / kStages) & 1u);
        const SlotMeta<E, Key> m = st.meta[slot];
        const unsigned char* data = ring + static_cast<size_t>(slot) * kTileBytes;
        int vote;
        int r = consume_tile<Key, MIN, FILTER>(data, m.par, m.tlen, m.lbase, buf, &st.cnt, K,
                                               flush_soft, &vote);
        bool deferred = r < 0;
        if (!deferred) {
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[slot]);
        }
        while (cbar_or(vote != 0)) {
            flush<Key, MIN>(buf, &st, hdr, k, K);
            vote = 0;
            if (deferred) {  // redo this warp's part of the tile with the new bound
                const E tau = better(st.tau, m.par.tau) ? st.tau : m.par.tau;
                const Par<E, Key> pr = make_par<Key, MIN>(tau);
                r = consume_tile<Key, MIN, FILTER>(data, pr, m.tlen, m.lbase, buf, &st.cnt, K,
                                                   flush_soft, &vote);
                deferred = r < 0;
                if (!deferred) {
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&empty[slot]);
                }
            }
        }
    }
    CSync::sync();
    if (st.cnt > 0) flush<Key, MIN>(buf, &st, hdr, k, K);

    // ---- hand the CTA's top-k to the reduction (last CTA to arrive) ----
    GBuf<E> cand;
    cand.init(p.ws + sizeof(WsHeader), static_cast<size_t>(G) * k);
    if (G > 1) {
        for (int j = tid; j < k; j += kNC) cand.st(static_cast<size_t>(c) * k + j, buf.ld(j));
        __threadfence();
        CSync::sync();
        if (tid == 0) st.last = (atomicAdd(&hdr->ticket, 1u) == G - 1u) ? 1 : 0;
        CSync::sync();
        if (!st.last) return;
        __threadfence();
        // Candidates of every other CTA that can still be in the top-k: e >= tau_g
        // (tau_g is some CTA's k-th best, so anything worse has k better entries).
        const E tg = tau_from_raw<E>(tau_load_raw(hdr));
        const size_t total = static_cast<size_t>(G) * k;
        constexpr int CI = 8;  // entries per thread per chunk
        constexpr int CH = CI * kNC;
        for (size_t q0 = 0; q0 < total; q0 += CH) {
            E ents[CI];
            uint32_t mask = 0;
#pragma unroll
            for (int r = 0; r < CI; ++r) {
                const size_t q = q0 + tid + static_cast<size_t>(r) * kNC;
                ents[r] = E::sentinel();
                if (q < total && q / k != c) {
                    const E e = cand.ld(q);
                    if (!e.is_sentinel() && !better(tg, e)) {
                        ents[r] = e;
                        mask |= 1u << r;
                    }
                }
            }
            bool deferred = true;
            while (true) {
                int vote = 0;
                if (deferred) {
                    int after = 0;
                    if (__any_sync(0xFFFFFFFFu, mask != 0u)) {
                        const int old = append<E, CI>(buf, &st.cnt, ents, mask, K, &after);
                        deferred = old < 0;
                        vote = deferred ? 1 : 0;
                    } else {
                        deferred = false;
                    }
                }
                if (!cbar_or(vote != 0)) break;
                flush<Key, MIN>(buf, &st, hdr, k, K);
            }
        }
        CSync::sync();
        if (st.cnt > 0) flush<Key, MIN>(buf, &st, hdr, k, K);
    }
    // ---- finalize: best first, original key bits, global index, payload ----
    for (int j = tid; j < k; j += kNC) {
        const E e = buf.ld(j);
        const uint32_t row = e.lidx();
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(p.base + row);
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = keys[row];
        if (p.out_payload) p.out_payload[j] = p.payload[row];
    }
    if (tid == 0) {  // leave the workspace zeroed for the next call
        hdr->tau_g = 0ull;
        hdr->ticket = 0u;
    }
}

template <class Key>
constexpr size_t select_smem_bytes() {
    return static_cast<size_t>(kStages) * kTileBytes +
           static_cast<size_t>(kCap) * SBuf<typename KeyTraits<Key>::E>::kBytes +
           static_cast<size_t>(2 * kStages) * 8;
}

}  // namespace topk
