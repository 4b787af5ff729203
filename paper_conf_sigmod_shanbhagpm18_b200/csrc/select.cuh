// select.cuh -- the fused streaming pass of bitonic top-k.
//
// One persistent CTA per SM reads its share of the input from HBM exactly once (1-D
// bulk TMA into a shared-memory ring), keeps the keys that can still be in the top-k,
// and runs the paper's local sort / merge / rebuild network (wnet.cuh, network.cuh)
// over the kept keys together with its running top-K run.  The last CTA to finish
// reduces all CTAs' runs and writes the result.  This is the paper's "SortReducer,
// then BitonicReducer until k remain" fused into one launch: the
// intermediate candidates live on chip / in L2, never in a second HBM pass.
//
// CTA = 15 consumer warps + 1 producer warp (16 warps: 4 per SM sub-partition, so a
// thread may use 128 registers).
//   * Producer warp: claims blocks of tiles from a global counter (fast SMs take more),
//     visits waves of blocks in a fixed pseudo-random order -- all SMs stream one
//     address window at a time (DRAM row locality) while no input order (sorted,
//     reversed) lines up with the scan, keeping the robustness the paper claims for
//     the pure method -- and issues one bulk copy per ring slot.
//   * Consumers: per key one compare against the threshold key t (fast test, a
//     superset of "can still be in the top-k"); for the few passing keys the exact
//     entry test and a warp-aggregated append into the survivor buffer -- the paper's
//     "buffer filler": a prefix sum of matches into a shared-memory buffer,
//     with the predicate "better than the current bound".
//   * When an append does not fit, the warp requests a collective flush: bitonic
//     top-K of [running run | survivors | sentinel padding].  No per-tile barrier: the
//     other warps join at their next wait point (tile wait or final drain); the
//     requesting warp keeps its ring slot and redoes its share of the tile afterwards.
//   * The bound: the CTA's own k-th best, every other CTA's k-th best (tau_g), and a
//     rank bound over every CTA's published run samples (the 2^j-th best of each run):
//     if t runs have a 2^j-th best >= v, then >= t * 2^j entries are >= v, so the t-th
//     largest sample of row j, t = ceil(k / 2^j), bounds the global k-th best.  All
//     bounds are entries owned by some run, so a strict test against them never drops
//     a top-k entry.
#pragma once
#include "cnet.cuh"
#include "keys.cuh"
#include "network.cuh"
#include "ptx.cuh"
#include "wnet.cuh"

#include <type_traits>

namespace topk {

#ifndef TOPK_VEC_PER_THREAD
#define TOPK_VEC_PER_THREAD 4
#endif
#ifndef TOPK_STAGES
#define TOPK_STAGES 5
#endif
#ifndef TOPK_FINAL_CODE_MIN
#define TOPK_FINAL_CODE_MIN 1025  // measured: k = 256 365.2 -> 362.5 us, increasing 366 -> 359 us
#endif
// Rows per consumer thread of a query-form stage (one TMA slab per column): larger slabs
// stream better -- KKKV (12-byte rows) 4 -> 8 rows: 820 -> 584 us (3 x 15 KB slabs per
// stage); key + WHERE column (8-byte rows) 8 -> 16: query 1 418 -> 391 us (KKV keeps 8:
// 394 -> 414 with 16)
#ifndef TOPK_ROW12_ITEMS
#define TOPK_ROW12_ITEMS 8
#endif
#ifndef TOPK_ROW8_ITEMS
#define TOPK_ROW8_ITEMS 16
#endif
#ifndef TOPK_FLUSH_ROWS
#define TOPK_FLUSH_ROWS 2  // A/B: 3 -> 2 rows: k=256 362.5 -> 360.5 us, few-distinct 399 -> 394 (1 row: ties 1.5x slower)
#endif
#ifndef TOPK_BOOT_LP
#define TOPK_BOOT_LP 1  // boot flush of a bag smaller than k: rank only as deep as the rank rows
#endif
#ifndef TOPK_BOOT_SMALL_K
#define TOPK_BOOT_SMALL_K 256  // K from which the boot buffer is kCap / 8 entries (else kCap)
#endif
#ifndef TOPK_BOOT_SAMPLE_Q
#define TOPK_BOOT_SAMPLE_Q 1  // ... also for the query forms (rows passing the WHERE)
#endif
#ifndef TOPK_BOOT_SAMPLE_E96
#define TOPK_BOOT_SAMPLE_E96 1  // ... also for three compound keys (KKKV)
#endif
#ifndef TOPK_BOOT_WAIT_KMIN
#define TOPK_BOOT_WAIT_KMIN 512  // K from which the boot flush waits for every CTA's samples
#endif
#ifndef TOPK_BOOT_SAMPLE
#define TOPK_BOOT_SAMPLE 1  // boot bag = the best key of each consumer thread's share of tile 0
#endif
#ifndef TOPK_ADAPTIVE_ORDER
#define TOPK_ADAPTIVE_ORDER 1
#endif
#ifndef TOPK_TAIL_ROWS
#define TOPK_TAIL_ROWS 3
#endif
#ifndef TOPK_LIMIT2
#define TOPK_LIMIT2 1024  // bag limit between the boot flush and the second flush
#endif
#ifndef TOPK_REFRESH_AT
#define TOPK_REFRESH_AT 12  // tile index at which warp 0 requests a rank-bound refresh
#endif
#ifndef TOPK_REFRESH_AT_NOWAIT
#define TOPK_REFRESH_AT_NOWAIT 6  // ... when the boot flush did not wait for its peers
#endif

constexpr int kNC = 480;                                    // consumer threads (15 warps)
constexpr int kNT = kNC + 32;                               // + one producer warp
constexpr int kTileBytes = kNC * 16 * TOPK_VEC_PER_THREAD;  // 30 KB per TMA stage
constexpr int kStagesMax = TOPK_STAGES;
constexpr int kSmemBudget = 227 * 1024 - 3 * 1024;  // dynamic smem (227 KB opt-in - static)
constexpr int kCap = 4096;            // survivor buffer entries (incl. the running run)
constexpr int kPubRows = 11;          // published 2^j-th best for j <= 10 (k up to 2048)
constexpr int kGMax = 160;            // CTAs (>= SM count)
constexpr int kScratch = kPubRows * kGMax;  // shared: staged samples (u64)
using CSync = NamedSync<kNC>;

template <class Key>
struct Cfg {
    // 12-byte entries (E64: f64 and compound keys) leave room for one stage less
    // (16-byte entries, E96: three compound keys, two less)
    static constexpr int kStages =
        std::is_same<typename KeyTraits<Key>::E, E96>::value   ? TOPK_STAGES - 2
        : std::is_same<typename KeyTraits<Key>::E, E64>::value ? TOPK_STAGES - 1
                                                               : TOPK_STAGES;
    static constexpr int kTileKeys = kTileBytes / static_cast<int>(sizeof(Key));
    static constexpr int kVecPerThread = kTileBytes / 16 / kNC;
    static constexpr int kItems = kTileKeys / kNC;  // keys per consumer thread per tile
    static_assert(kItems <= 32, "mask width");
};

// Query forms (the paper's §5 database integration; R17/R18): the
// streamed row is more than the key column.  Q bits: kQPred -- a u32 predicate column
// (WHERE), kQRank -- a second f32 column b with the ranking function f = a + w * b
// (ORDER BY f), kQKey2 -- a second f32 key column b (Key = KK32: ORDER BY a, b).  A ring
// stage then holds one slab per column, TK rows each.
// kQKey3 -- a third f32 key column c (Key = KKK32: ORDER BY a, b, c; with kQKey2).
constexpr int kQPred = 1, kQRank = 2, kQKey2 = 4, kQKey3 = 8;
template <class Key, int Q>
struct QCfg {
    static constexpr int kRowBytes = static_cast<int>(sizeof(Key)) +
                                     ((Q & (kQRank | kQKey2)) ? 4 : 0) + ((Q & kQKey3) ? 4 : 0) +
                                     ((Q & kQPred) ? 4 : 0);
    static constexpr int kItems =
        Q == 0 ? Cfg<Key>::kItems
               : (kRowBytes <= 8 ? ((Q & kQKey2) ? 8 : TOPK_ROW8_ITEMS)
                                : (kRowBytes == 12 ? TOPK_ROW12_ITEMS : 4));
    static constexpr int kTileKeys = Q == 0 ? Cfg<Key>::kTileKeys : kNC * kItems;
    static constexpr int kVecPerThread = kItems / KeyTraits<Key>::kVec;
    static constexpr int kOffB = kTileKeys * static_cast<int>(sizeof(Key));  // column b
    static constexpr int kOffC = kOffB + ((Q & (kQRank | kQKey2)) ? kTileKeys * 4 : 0);  // key 3
    static constexpr int kOffP = kOffC + ((Q & kQKey3) ? kTileKeys * 4 : 0);  // predicate
    static_assert(Q == 0 || kTileKeys * kRowBytes <= 2 * kTileBytes, "stage size");
    // ring: a query stage is TK rows of every column (<= one plain stage), so the ring
    // budget of the plain form holds more of them (up to kStagesMax)
    static constexpr int kSlotBytes = Q == 0 ? kTileBytes : (kTileKeys * kRowBytes + 127) / 128 * 128;
    // query forms: as many stages as fit next to the buffer, the sample scratch and the
    // code network (bytes in flight: a KKKV stage is only 23 KB), up to kStagesMax
    using E_ = typename KeyTraits<Key>::E;
    static constexpr int kOther = kCap * SBuf<E_>::kBytes + kScratch * 8 +
                                  (kCap / 512) * 512 * static_cast<int>(sizeof(typename CodeOf<E_>::C)) +
                                  2 * kStagesMax * 8;
    static constexpr int kFit = (kSmemBudget - kOther) / kSlotBytes;
    static constexpr int kStages =
        Q == 0 ? Cfg<Key>::kStages : (kFit < kStagesMax ? kFit : kStagesMax);
    static_assert(kStages >= 2, "ring");
    static_assert(kTileKeys % 4 == 0, "TMA sizes are multiples of 16 bytes");
};

struct WsHeader {
    unsigned long long tau_g;  // max over CTAs of their k-th best
    unsigned int ticket;       // CTAs finished
    unsigned int next_tile;    // dynamic work claiming counter
    unsigned int npub;         // CTAs that published their boot-flush samples
    unsigned int pad[11];
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
    uint32_t perm_h;   // Feistel half-width (bits) over nwaves; 0 = identity order
    uint32_t blk;      // tiles per claimed block
    uint32_t nblocks;  // ceil(ntiles / blk)
    uint32_t wave;     // blocks per wave (permutation unit)
    uint32_t nwaves;   // ceil(nblocks / wave)
    uint32_t gmax;     // workspace layout: published-sample columns (>= gridDim.x)
    uint32_t J;        // published samples per CTA: the 2^j-th best of its run, j < J
    // query forms (Q != 0; select_kernel's template argument)
    const float* col_b;    // kQRank: column b of f = key + rank_w * b; kQKey2: second key
    float* out_keys2;      // kQKey2: b of each result row
    uint32_t order2_min;   // kQKey2: b ascending (1) or descending (0)
    const float* col_c;    // kQKey3: third key column
    float* out_keys3;
    uint32_t order3_min;
    const uint32_t* pred;  // kQPred: predicate column
    float rank_w;
    uint32_t pred_in;      // 1: membership (pred < 64 and bit pred of pred_mask); 0: range
    uint32_t pred_lo;      // range: pred_lo <= pred < pred_lo + pred_span
    uint32_t pred_span;
    uint64_t pred_mask;
};

// WHERE (reading R17): range lo <= v < lo + span as one unsigned compare, or IN-list
// membership over dictionary codes < 64.
__device__ __forceinline__ bool pred_ok(const SelectParams& p, uint32_t v) {
    const bool in = v < 64u && ((p.pred_mask >> (v & 63u)) & 1ull);
    const bool rg = v - p.pred_lo < p.pred_span;
    return p.pred_in ? in : rg;
}
// ORDER BY f (reading R18): f = a + w * b, the product and the sum each rounded to
// nearest f32 (no fused multiply-add, so the oracle's plain C arithmetic agrees).
// A NaN result is returned as the canonical quiet NaN 0x7FC00000 (IEEE-754 leaves a
// computed NaN's payload open; the order code of every NaN is the same).
__device__ __forceinline__ float rank_f(float a, float w, float b) {
    const float f = __fadd_rn(a, __fmul_rn(w, b));
    return f != f ? __uint_as_float(0x7FC00000u) : f;
}

// Workspace: [WsHeader | pub: u64[kPubRows][gmax] | cand: G x k entries]
__host__ __device__ constexpr size_t ws_pub_offset() { return 64; }
__host__ __device__ inline size_t ws_cand_offset(uint32_t gmax) {
    return 64 + static_cast<size_t>(kPubRows) * gmax * 8;
}

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

template <>
struct GBuf<E96> {
    uint64_t* c;
    uint32_t* c3;
    uint32_t* ni;
    __device__ __forceinline__ void init(unsigned char* base, size_t cap) {
        c = reinterpret_cast<uint64_t*>(base);
        c3 = reinterpret_cast<uint32_t*>(base + 8 * cap);
        ni = reinterpret_cast<uint32_t*>(base + 12 * cap);
    }
    __device__ __forceinline__ E96 ld(size_t i) const {
        return E96{__ldcg(c + i), __ldcg(c3 + i), __ldcg(ni + i)};
    }
    __device__ __forceinline__ void st(size_t i, E96 e) const {
        __stcg(c + i, e.c);
        __stcg(c3 + i, e.c3);
        __stcg(ni + i, e.ni);
    }
};

// Bounds as 64-bit words: E32 the packed entry (exact, index included); E64 the code
// only, read back as {code, ni = 0} -- i.e. non-strict on that code (still valid).
__device__ __forceinline__ unsigned long long bound_word(E32 e) { return e.v; }
__device__ __forceinline__ unsigned long long bound_word(E64 e) { return e.c; }
__device__ __forceinline__ unsigned long long bound_word(E96 e) { return e.c; }
template <class E>
__device__ __forceinline__ E from_bound_word(unsigned long long w);
template <>
__device__ __forceinline__ E32 from_bound_word<E32>(unsigned long long w) { return E32{w}; }
template <>
__device__ __forceinline__ E64 from_bound_word<E64>(unsigned long long w) { return E64{w, 0u}; }
template <>
__device__ __forceinline__ E96 from_bound_word<E96>(unsigned long long w) { return E96{w, 0u, 0u}; }
__device__ __forceinline__ void tau_publish(WsHeader* h, E32 e) { atomicMax(&h->tau_g, e.v); }
__device__ __forceinline__ void tau_publish(WsHeader* h, E64 e) { atomicMax(&h->tau_g, e.c); }
__device__ __forceinline__ void tau_publish(WsHeader* h, E96 e) { atomicMax(&h->tau_g, e.c); }

__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
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

// Bijection on [0, n): 4-round Feistel on 2h bits with cycle walking.
__device__ __forceinline__ uint32_t feistel_perm(uint32_t i, uint32_t n, uint32_t h) {
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
            const uint32_t nl = R;
            R = L ^ (f & mask);
            L = nl;
        }
        x = (L << h) | R;
    } while (x >= n);
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

constexpr uint32_t kEndTile = 0xFFFFFFFFu;
constexpr int kReqFlush = 1, kReqRefresh = 2, kReqBoot = 4;

// Shared state of one CTA.
template <class E, class Key>
struct CtaState {
    int cnt;                   // bag entries buf[0 .. cnt) (reservations; see reserve())
    int cnt_fail;              // min start of a failed reservation (INT_MAX: none); = cnt + 1
    int req;                   // collective requests (kReqFlush | kReqRefresh)
    int nflush;                // flushes done
    int last;                  // this CTA reduces all candidates
    unsigned long long tau_w;  // E32: the bound as one packed word
    E tau;                     // E64: the bound
    Par<E, Key> par;           // E64: fast-test parameters of tau
    int sorted_cnt;            // cnt right after the last exact flush (bag still sorted), else -1
    int pubd;                  // this CTA counted itself in WsHeader::npub
    int cnt_run;               // real entries in the CTA's final run buf[0 .. K)
    int limit;                 // bag capacity until the next flush
    int ties;                  // a code-path stream flush could not shrink the bag
    int wcnt[16];              // compaction: kept entries per consumer warp
    unsigned long long own_w;  // the bag's own k-th best as a bound word (0 = none)
    unsigned long long best[kPubRows];
    int npres[kPubRows];       // rank_rows: present samples per ranked row
    int perm_mode;             // wave order: 0 undecided, 1 address, 2 permuted, 3 backwards
    int nx;                    // kBoot, CTA 0: extras kept aside until the boot flush
    E xent[8];
    uint32_t tile[kStagesMax];  // tile id of each ring slot (producer); kEndTile = done
};

// Current bound / raise it (thread 0 inside a collective).
template <class Key>
__device__ __forceinline__ E32 bound_get(const CtaState<E32, Key>& st) { return E32{st.tau_w}; }
template <class Key>
__device__ __forceinline__ E64 bound_get(const CtaState<E64, Key>& st) { return st.tau; }
template <class Key>
__device__ __forceinline__ E96 bound_get(const CtaState<E96, Key>& st) { return st.tau; }
template <class Key, bool MIN>
__device__ __forceinline__ void bound_set(CtaState<E32, Key>* st, E32 t) {
    if (t.v > st->tau_w) st->tau_w = t.v;
}
template <class Key, bool MIN>
__device__ __forceinline__ void bound_set(CtaState<E64, Key>* st, E64 t) {
    if (better(t, st->tau)) {
        st->tau = t;
        st->par = make_par<Key, MIN>(t);
    }
}
template <class Key, bool MIN>
__device__ __forceinline__ void bound_set(CtaState<E96, Key>* st, E96 t) {
    if (better(t, st->tau)) {
        st->tau = t;
        st->par = make_par<Key, MIN>(t);
    }
}
// Lower the bound by one entry step (the boot sample's re-read tile: keys >= the old bound
// pass the strict test against the new one).  Thread 0 inside a collective.
template <class Key, bool MIN>
__device__ __forceinline__ void bound_weaken1(CtaState<E32, Key>* st) {
    if (st->tau_w != 0ull) st->tau_w -= 1ull;
}
template <class Key, bool MIN>
__device__ __forceinline__ void bound_weaken1(CtaState<E64, Key>* st) {
    E64 t = st->tau;
    if (t.is_sentinel()) return;
    if (t.ni != 0u) {
        t.ni -= 1u;
    } else {
        t.c -= 1ull;
        t.ni = 0xFFFFFFFFu;
    }
    st->tau = t;
    st->par = make_par<Key, MIN>(t);
}
template <class Key, bool MIN>
__device__ __forceinline__ void bound_weaken1(CtaState<E96, Key>* st) {
    E96 t = st->tau;
    if (t.is_sentinel()) return;
    // (c, c3, ni) lexicographic: subtract one from the 128-bit word with borrows
    if (t.ni != 0u) {
        t.ni -= 1u;
    } else {
        t.ni = 0xFFFFFFFFu;
        if (t.c3 != 0u) {
            t.c3 -= 1u;
        } else {
            t.c3 = 0xFFFFFFFFu;
            t.c -= 1ull;
        }
    }
    st->tau = t;
    st->par = make_par<Key, MIN>(t);
}

// The bound a consumer uses for one tile (changes only inside collectives).
template <class Key, bool MIN>
__device__ __forceinline__ Par<E32, Key> load_par(const CtaState<E32, Key>& st) {
    return make_par<Key, MIN>(E32{st.tau_w});
}
template <class Key, bool MIN>
__device__ __forceinline__ Par<E64, Key> load_par(const CtaState<E64, Key>& st) {
    return st.par;
}
template <class Key, bool MIN>
__device__ __forceinline__ Par<E96, Key> load_par(const CtaState<E96, Key>& st) {
    return st.par;
}

// Reserve `total` buffer entries (lane 31 of a warp): one atomicAdd, or -1 if they
// did not fit under `limit`.  A failure is NOT undone (add-then-undo is racy: with two
// failed adds in flight, undoing one lets a third warp succeed ABOVE the other's phantom
// entries -- a hole of stale entries in the bag (duplicates) and entries past the count
// (lost); seen as ~4% wrong answers at f64, 2^24 keys, k = 1024).  Instead the counter
// stays monotone until the flush, so the reservations are ordered by `old`: every one
// after the first failure F starts at >= old_F + total_F > limit and fails too, every
// one before F succeeded, and they fill exactly [0, old_F).  A failure records its
// `old` in cnt[1] (CtaState::cnt_fail, atomicMin); the flush that every failure leads
// to takes min(cnt, cnt_fail) as the bag size (bag_count()) and resets both.
__device__ __forceinline__ int reserve(int* cnt, int total, int limit) {
#ifdef TOPK_RESERVE_CAS  // (dev A/B: compare-and-swap form, ~10 us slower at k = 256)
    int old = *reinterpret_cast<volatile int*>(cnt);
    while (old + total <= limit) {
        const int seen = atomicCAS(cnt, old, old + total);
        if (seen == old) return old;
        old = seen;
    }
    return -1;
#else
    const int old = atomicAdd(cnt, total);
    if (old + total <= limit) return old;
    atomicMin(cnt + 1, old);
    return -1;
#endif
}

// Warp-aggregated append of ITEMS candidate entries per thread (mask = which).
// Returns the count before this warp's entries, or -1 if they did not fit.
template <class E, int ITEMS>
__device__ __forceinline__ int append(const SBuf<E>& buf, int* s_cnt, const E (&ents)[ITEMS],
                                      uint32_t mask, int limit) {
    const int lane = threadIdx.x & 31;
    const int cnt = __popc(mask);
    int incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    const int total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    if (total == 0) return 0;
    int old = 0;
    if (lane == 31) old = reserve(s_cnt, total, limit);
    old = __shfl_sync(0xFFFFFFFFu, old, 31);
    if (old < 0) return -1;
    int w = old + incl - cnt;
#pragma unroll
    for (int q = 0; q < ITEMS; ++q)
        if ((mask >> q) & 1u) buf.st(w++, ents[q]);
    return old;
}

// Debug instrumentation, compiled only into -DTOPK_DEBUG builds (tools/, variant
// builds through _build.build(extra_flags=[...])); the product library has none of it.
//  * g_stats: whole-launch counters read with topk_debug_stats(): [0] flushes,
//    [1] survivors flushed, [2] flush cycles (thread 0), [3] deferrals, [4] tiles
//    consumed, [5] refreshes, [6] exact flushes, [7] sentinel outputs (a bug).
//  * g_trace: per CTA up to 62 (event << 56 | globaltimer ns) stamps written by consumer
//    thread 0 (1 start, 2/3 flush begin/end, 4 stream end, 5 tail begin, 6 end,
//    7 refresh); g_trace[c][0] = count.  Enabled by c_trace_on.
//  * c_dbg: knobs (topk_debug_flags): bit 0 -- no code-network path; bit 1 -- no
//    boot-time wait for peers; bit 2 -- no early second flush; bit 3 -- no small-buffer
//    exact network; bits 4-5 -- rank-bound rows (0 = 3); bits 6-7 -- second-flush limit
//    512 * (1 + v); bits 8-10 -- boot buffer kCap >> v (0 = by K).
constexpr int kTraceCtas = 160, kTraceLen = 64;
#ifdef TOPK_DEBUG
static __device__ unsigned long long g_stats[8];  // per translation unit (select_inst.cuh)
static __device__ unsigned long long g_trace[kTraceCtas][kTraceLen];
static __device__ __constant__ int c_trace_on;
static __device__ __constant__ int c_dbg_sym;  // topk_debug_flags
#ifdef TOPK_LIGHT  // -DTOPK_DEBUG -DTOPK_LIGHT: trace stamps only (no counters, no knobs)
constexpr int c_dbg = 0;
#else
#define c_dbg c_dbg_sym
#endif
#if defined(TOPK_DUPCHECK) || defined(TOPK_LIGHT)
#define TOPK_STAT(i, v) ((void)0)
#else
#define TOPK_STAT(i, v) atomicAdd(&g_stats[i], static_cast<unsigned long long>(v))
#endif
__device__ __forceinline__ void trace(int ev) {
    if (!c_trace_on || blockIdx.x >= kTraceCtas) return;
    // stamps are SM clock cycles (a %globaltimer read costs ~1 us and inflated every
    // interval it bracketed); the CTA's first stamp also records (globaltimer, clock)
    // in the last two slots, which align the CTAs (tools/trace.py)
    const unsigned long long t = clock64();
    unsigned long long* row = g_trace[blockIdx.x];
    __shared__ int s_trace_n;
    if (ev == 1) {
        s_trace_n = 0;
        unsigned long long g;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g));
        row[kTraceLen - 1] = g;
        row[kTraceLen - 2] = t;
    }
    const int n = s_trace_n;
    if (n + 3 < kTraceLen) {
        row[n + 1] = (static_cast<unsigned long long>(ev) << 56) | (t & 0x00FFFFFFFFFFFFFFull);
        row[0] = static_cast<unsigned long long>(n + 1);
        s_trace_n = n + 1;
    }
}
#else
constexpr int c_dbg = 0;
#define TOPK_STAT(i, v) ((void)0)
__device__ __forceinline__ void trace(int) {}
#endif

// Everything a collective needs besides the buffer.
struct Ctx {
    WsHeader* hdr;
    unsigned long long* pub;      // global [kPubRows][gmax]
    unsigned long long* scratch;  // shared [J][G]
    int k, K;
    int G, gmax, J;
    int j_lo, nrows;  // rank-bound rows used: j_lo .. j_lo + nrows - 1 (t <= G)
    int Lp;           // code network size log2 K' (K' = min(max(K, 16), 512)); -1: not used
    void* codes;      // shared: code-network scratch (8 x K' codes)
    bool filter;
    int boot_l2;      // kBoot: bag limit of the second flush (0: no boot sample)
    bool boot_wait;   // the boot flush waits (<= 20 us) until every CTA published samples
};

// Sample rows in shared scratch: row r at scratch + r * ScrStride(G) (padded with zeros
// to a multiple of 4 words: 16-byte loads, 2 per step).
__device__ __forceinline__ int scr_stride(int G) { return (G + 3) & ~3; }

// Rank bound over scratch rows (row r = sample row j_lo + r; 0 = missing sample): the
// t-th largest word x_t of row j, t = ceil(k / 2^j) <= G, if it is not missing.  Only
// the nrows (<= 3) rows with the smallest valid j are ranked -- they give the tightest
// bounds (a deeper row samples a weaker quantile of every run).  When the row has at
// least t present samples, x_t = the smallest present word v with #{x > v} <= t - 1
// (every v >= x_t has at most t - 1 larger words, every v < x_t has x_1 .. x_t above
// it); with fewer, there is no bound.  One thread per word counts the strictly larger
// ones (16-byte loads, four independent counters -- the dependent one-counter loop took
// ~3.4 us at G = 148, latency-bound), the qualifying words meet in a shared atomicMin,
// the present words are counted per row.  Collective (consumers); st->best[] gets one
// word per ranked row, 0 elsewhere (thread 0 finishes it: only thread 0 reads
// st->best).  Entry: scratch filled and barrier passed; exit: after a barrier.
template <class E, class Key>
__device__ void rank_rows(CtaState<E, Key>* st, const Ctx& cx) {
    static_assert(3 * kGMax <= kNC, "one ranked word per consumer thread");
    if (threadIdx.x < kPubRows) {
        st->best[threadIdx.x] = ~0ull;
        st->npres[threadIdx.x] = 0;
    }
    CSync::sync();
    if (threadIdx.x == 0) trace(23);
    const int S = scr_stride(cx.G);
    const int q = threadIdx.x;  // nrows * G <= 3 * kGMax <= kNC: one pass
    const int r = q / cx.G, cc = q - r * cx.G;
    const bool in = r < cx.nrows;
    const unsigned long long* row = cx.scratch + (in ? r : 0) * S;
    const unsigned long long v = in ? row[cc] : 0ull;
    const int ji = cx.j_lo + r;
    if (v != 0ull) {
        const int t = (cx.k + (1 << ji) - 1) >> ji;
        const ulonglong2* row2 = reinterpret_cast<const ulonglong2*>(row);
        int g0 = 0, g1 = 0, g2 = 0, g3 = 0;
#pragma unroll 4
        for (int c2 = 0; c2 < S / 2; c2 += 2) {
            const ulonglong2 a = row2[c2], b = row2[c2 + 1];
            g0 += a.x > v ? 1 : 0;
            g1 += a.y > v ? 1 : 0;
            g2 += b.x > v ? 1 : 0;
            g3 += b.y > v ? 1 : 0;
        }
        if (g0 + g1 + g2 + g3 <= t - 1) atomicMin(&st->best[ji], v);
    }
    {   // present samples per row: one shared atomic per (warp, row)
        const uint32_t same = __match_any_sync(0xFFFFFFFFu, in ? r : -1);
        const uint32_t pres = __ballot_sync(0xFFFFFFFFu, v != 0ull);
        const int lane = threadIdx.x & 31;
        if (in && lane == __ffs(same) - 1) atomicAdd(&st->npres[ji], __popc(same & pres));
    }
    if (threadIdx.x == 0) trace(24);
    CSync::sync();
    if (threadIdx.x == 0)
        for (int j2 = 0; j2 < kPubRows; ++j2) {
            const int t = (cx.k + (1 << j2) - 1) >> j2;
            if (st->best[j2] == ~0ull || st->npres[j2] < t) st->best[j2] = 0ull;
        }
}

// Load every CTA's published samples of the ranked rows into shared scratch (stale
// values are smaller, still valid).
__device__ __forceinline__ void load_pub(const Ctx& cx) {
    const int S = scr_stride(cx.G);
    const int RS = cx.nrows * S;
    for (int q = threadIdx.x; q < RS; q += kNC) {
        const int r = q / S, cc = q - r * S;
        cx.scratch[q] = cc < cx.G ? ld_relaxed_u64(reinterpret_cast<const uint64_t*>(
                                        cx.pub + static_cast<size_t>(cx.j_lo + r) * cx.gmax + cc))
                                  : 0ull;
    }
}

// Fold st->best[] (and tau_g, and the run's own k-th best) into the CTA bound.
template <class Key, bool MIN>
__device__ __forceinline__ void fold_bounds(CtaState<typename KeyTraits<Key>::E, Key>* st,
                                            const Ctx& cx, typename KeyTraits<Key>::E own) {
    using E = typename KeyTraits<Key>::E;
    E tau = bound_get(*st);
    if (!own.is_sentinel() && better(own, tau)) tau = own;
    const E tg =
        from_bound_word<E>(ld_relaxed_u64(reinterpret_cast<const uint64_t*>(&cx.hdr->tau_g)));
    if (better(tg, tau)) tau = tg;
    for (int ji = 0; ji < cx.J; ++ji) {
        const E b = from_bound_word<E>(st->best[ji]);
        if (st->best[ji] != 0ull && better(b, tau)) tau = b;
    }
    bound_set<Key, MIN>(st, tau);
}

#ifdef TOPK_DUPCHECK
// (dev) count duplicate row ids in buf[0 .. cnt) into g_stats[slot]; order violations of
// a sorted prefix into g_stats[oslot] (collective)
template <class E>
__device__ void dbg_check(const SBuf<E>& buf, int cnt, int slot, int sorted_n, int oslot) {
    CSync::sync();
    unsigned long long d = 0, o = 0;
    for (int i = threadIdx.x; i < cnt; i += kNC) {
        const E a = buf.ld(i);
        if (a.is_sentinel()) continue;
        for (int j = i + 1; j < cnt; ++j) {
            const E b = buf.ld(j);
            if (!b.is_sentinel() && b.lidx() == a.lidx()) ++d;
        }
        if (i + 1 < sorted_n && better(buf.ld(i + 1), a)) ++o;
    }
    if (d) atomicAdd(&g_stats[slot], d);
    if (o) atomicAdd(&g_stats[oslot], o);
    CSync::sync();
}
#define TOPK_DUP(...) dbg_check(__VA_ARGS__)
static __device__ unsigned int g_tiles[1 << 16];
#else
#define TOPK_DUP(...) ((void)0)
#endif

enum FlushMode { kFlushStream = 0, kFlushFinal = 1 };

// A code as a bound word (the weakest entry with that code: index "infinity"), i.e. a
// NON-strict bound on the code -- valid whenever >= r entries have code >= c.
template <class E>
__device__ __forceinline__ unsigned long long code_word(typename CodeOf<E>::C c);
template <>
__device__ __forceinline__ unsigned long long code_word<E32>(uint32_t c) {
    return static_cast<unsigned long long>(c) << 32;
}
template <>
__device__ __forceinline__ unsigned long long code_word<E64>(uint64_t c) {
    return c;
}
template <>
__device__ __forceinline__ unsigned long long code_word<E96>(uint64_t c) {
    return c;
}

__device__ __forceinline__ unsigned long long global_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
constexpr unsigned long long kBootWaitNs = 20000;  // cap of the boot-time wait for peers

// Bound round (collective; entry after the caller's samples were stored, exit after a
// barrier):  stream mode -- publish the bag's k-th best (tau_g), at the first flush wait
// (bounded) until every CTA published its samples, then the rank bound over all CTAs'
// samples;  every mode -- thread 0 folds own / tau_g / rank rows into the CTA bound.
template <class Key, bool MIN>
__device__ void take_bounds(CtaState<typename KeyTraits<Key>::E, Key>* st, const Ctx& cx,
                            typename KeyTraits<Key>::E own, bool publish) {
    if (publish) {
        if (threadIdx.x == 0 && !own.is_sentinel()) tau_publish(cx.hdr, own);
        if (cx.boot_wait && !st->pubd && cx.G > 1 && !(c_dbg & 2)) {
            // boot: every CTA flushes its first buffer at about the same time; wait for
            // their samples so the very first bound is the cross-CTA rank bound (a stale
            // or missing sample only weakens the bound -- the wait is a performance
            // matter, never a correctness one)
            CSync::sync();
            if (threadIdx.x == 0) {
                atomicAdd(&cx.hdr->npub, 1u);
                st->pubd = 1;
                const unsigned long long t0 = global_ns();
                while (ld_relaxed_u32(&cx.hdr->npub) < static_cast<uint32_t>(cx.G) &&
                       global_ns() - t0 < kBootWaitNs)
                    __nanosleep(64);
                __threadfence();
            }
            CSync::sync();
        }
        // stream flushes rank TOPK_FLUSH_ROWS sample rows (the tail ranks all nrows)
        Ctx cr = cx;
        if (cr.nrows > TOPK_FLUSH_ROWS) cr.nrows = TOPK_FLUSH_ROWS;
        load_pub(cr);
        CSync::sync();
        if (threadIdx.x == 0) trace(21);
        rank_rows(st, cr);
        if (threadIdx.x == 0) trace(22);
    }
    if (threadIdx.x == 0) {
        if (!publish)
            for (int ji = 0; ji < kPubRows; ++ji) st->best[ji] = 0ull;
        if (cx.filter) fold_bounds<Key, MIN>(st, cx, own);
        // (no boot wait: the first publishing flush still ends the boot; every read of
        // pubd for this flush is behind us)
        if (publish) st->pubd = 1;
    }
    CSync::sync();
}

// Keep only the bag entries not worse than tau (collective).  Every entry is read into
// registers before a barrier, then written compacted to the front (order is
// irrelevant: the bag is unordered).  Returns the new count (in every thread).
template <class E>
__device__ int compact_bag(const SBuf<E>& buf, int cnt, E tau, int* s_w) {
    constexpr int RC = (kCap + kNC - 1) / kNC;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    E ents[RC];
    uint32_t keep = 0;
#pragma unroll
    for (int q = 0; q < RC; ++q) {
        const int e = tid + q * kNC;
        ents[q] = e < cnt ? buf.ld(e) : E::sentinel();
        // keep e >= tau: tau may be an entry of this very bag (its own k-th best, or
        // its own published sample coming back through tau_g / the rank rows), and
        // that entry can be the global k-th best
        if (e < cnt && !better(tau, ents[q])) keep |= 1u << q;
    }
    const int c = __popc(keep);
    int incl = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) s_w[w] = incl;
    CSync::sync();
    int off = 0, all = 0;
#pragma unroll
    for (int v = 0; v < kNC / 32; ++v) {
        const int x = s_w[v];
        off += v < w ? x : 0;
        all += x;
    }
    int pos = off + incl - c;
#pragma unroll
    for (int q = 0; q < RC; ++q)
        if ((keep >> q) & 1u) buf.st(pos++, ents[q]);
    CSync::sync();
    return all;
}

// Bag capacity after `nflush` flushes: right after the boot flush a small one, so that a
// cheap second flush soon publishes samples of many more keys (the boot samples cover
// one buffer per CTA only) and the rank bound tightens early.  A stream flush always
// leaves at most half of the next limit (progress: a warp appends <= 512 at a time).
#ifndef TOPK_L2_BOOT_MUL
#define TOPK_L2_BOOT_MUL 4
#endif
#ifndef TOPK_L2_BOOT_KMAX
#define TOPK_L2_BOOT_KMAX 256
#endif
__device__ __forceinline__ int next_limit(int nflush, int K, int Lp, int ties, int boot_l2 = 0) {
    // (K = 256: 512 measured 6 us faster than 1024, K = 128: 360 -> 354 us; other K: 512
    // no better, 2048 slower)
    const int l2 = (c_dbg >> 6) & 3 ? 512 * (1 + ((c_dbg >> 6) & 3))
                   : (K == 128 || K == 256) ? 512 : TOPK_LIMIT2;
    // Tie-heavy bags (the code path failed on equal keys) flush exactly at a small size:
    // every CTA meets the ties at about the same time and a 4096-entry exact flush idles
    // the HBM for ~20 us.  Progress: room for a warp's largest append (32 lanes x 16
    // keys = 512) on top of the K entries an exact flush keeps.
    if (ties) return max(max(2 * K, K + 512), kCap >> 3);
    // After a boot sample (boot_sample) the bound already stands on a 16x larger sample:
    // the survivors arrive ~16x slower, so the second flush -- the one that publishes
    // samples of many tiles -- comes at a much smaller bag (Ctx::boot_l2).  (Progress:
    // that flush makes nflush 2, whose limit is kCap.)
    if (boot_l2 > 0 && nflush == 1 && Lp >= 0 && !(c_dbg & 4)) return boot_l2;
    return (nflush == 1 && Lp >= 0 && !(c_dbg & 4)) ? max(l2, 2 * K) : kCap;
}

// Collective flush (consumers) of the candidate bag buf[0 .. cnt):
//   code path (filter mode, ranking min(K, 512) codes; every stream flush, and a final flush of a large
//     bag): the code-only network (cnet.cuh) gives the bag's k-th best code and its
//     2^j-th best codes -> publish, bound round, drop every entry worse than the new
//     bound.  A stream flush ends here unless ties kept the bag over half full.
//   exact path: bitonic top-K of [bag | sentinel padding] (wnet.cuh: local sort, merge,
//     rebuild on (code, index) entries) -> buf[0 .. K) best first; in stream mode its
//     exact samples / k-th best are published as well.
// Entry: barrier-consistent; exit: same.
template <class Key, bool MIN>
__device__ void flush(const SBuf<typename KeyTraits<Key>::E>& buf,
                      CtaState<typename KeyTraits<Key>::E, Key>* st, const Ctx& cx,
                      FlushMode mode) {
    using E = typename KeyTraits<Key>::E;
    using C = typename CodeOf<E>::C;
    const int k = cx.k, K = cx.K;
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int c = static_cast<int>(blockIdx.x);
    // (a failed reservation leaves cnt above the filled prefix; see reserve())
    int cnt = st->cnt < st->cnt_fail ? st->cnt : st->cnt_fail;
    [[maybe_unused]] const int cnt0 = cnt;
    if (threadIdx.x == 0) trace(2);
    [[maybe_unused]] const long long t0 = clock64();
    const bool publish = mode == kFlushStream && cx.filter;
    bool done = false;
    // (tie-heavy input -- a code bound cannot separate equal codes -- makes the code
    // path useless: after it failed once, stream flushes go straight to the exact path)
    // (a final flush of a bag the small exact network can take directly skips the code
    // network: TOPK_FINAL_CODE_MIN is the smallest such bag that still goes through it)
    const bool try_code = !st->ties && (publish || (cnt > 2 * K && K <= (1 << cx.Lp) &&
                                                    cnt >= TOPK_FINAL_CODE_MIN));
    bool tried = false;
    if (cx.filter && cx.Lp >= 0 && !(c_dbg & 1) && try_code) {
        tried = true;
        C* S = static_cast<C*>(cx.codes);
        // A boot bag smaller than k has no k-th best to publish: its flush only needs the
        // samples the first rank bound uses (rows j_lo .. j_lo + TOPK_FLUSH_ROWS - 1), so
        // the code network ranks only that deep (measured, 2^29 uniform: k = 1024 393 ->
        // 391 us, k = 2048 432 -> 420; a bag that holds k keeps the full depth: its k-th
        // best, published as tau_g, is what bounds sorted input early)
        int Lp = cx.Lp;
        if (TOPK_BOOT_LP && publish && !st->pubd && cnt < k) {
            const int deep = cx.j_lo + cx.nrows - 1;
            Lp = min(cx.Lp, max(4, deep));
        }
        cnet_topk_codes<E, kNC / 32, CSync>(buf, cnt, Lp, S, w, lane);
        if (threadIdx.x == 0) trace(16);
        const int Kp = 1 << Lp;  // codes the network ranked (S[0 .. Kp))
        if (publish && threadIdx.x < cx.J && threadIdx.x <= Lp && cnt >= (1 << threadIdx.x)) {
            st_relaxed_u64(cx.pub + static_cast<size_t>(threadIdx.x) * cx.gmax + c,
                           code_word<E>(S[(1 << threadIdx.x) - 1]));
            __threadfence();
        }
        // the bag's own k-th best code (only if the network ranked that far)
        const E own =
            (cnt >= k && k <= Kp) ? from_bound_word<E>(code_word<E>(S[k - 1])) : E::sentinel();
        // half of the top K' codes equal: heavy ties (few distinct keys), which a code
        // bound cannot separate -- finish exactly (strict (code, index) bound) at once
        const bool heavy = cnt >= Kp && S[Kp - 1] == S[Kp / 2 - 1];
        take_bounds<Key, MIN>(st, cx, own, publish);
        if (!heavy) cnt = compact_bag<E>(buf, cnt, bound_get(*st), st->wcnt);
        // a code bound that dropped less than half of a large bag is defeated by ties
        // (equal codes): finish exactly, and skip the code path from now on
        const bool weak = heavy || (cnt > 2 * K && 2 * cnt > cnt0);
        done = mode == kFlushStream && !weak &&
               cnt <= next_limit(st->nflush + 1, K, cx.Lp, 0, cx.boot_l2) / 2;
        // (the boot sample's bag is emptied after this flush: no exact pass unless the
        // code bound was defeated by ties)
        if (st->req & kReqBoot) done = !weak;
    }
    if (!done) {
        int P = next_pow2_i(cnt);
        if (P < 2 * K) P = 2 * K;
        if (P < 64) P = 64;
        for (int i = cnt + threadIdx.x; i < P; i += kNC) buf.st(i, E::sentinel());
        CSync::sync();
        if (P <= 512 && !(c_dbg & 8))
            wnet_small<E, 2, kNC / 32, CSync>(buf, P, __ffs(K) - 1, w, lane);
        else if (P <= 1024 && !(c_dbg & 8))
            wnet_small<E, 4, kNC / 32, CSync>(buf, P, __ffs(K) - 1, w, lane);
        else
            wnet_topk<E, kNC / 32, CSync>(buf, P, __ffs(K) - 1, w, lane);
        const E kth = buf.ld(k - 1);
        if (publish) {
            if (threadIdx.x < cx.J) {
                const E e = buf.ld((1 << threadIdx.x) - 1);
                if (!e.is_sentinel())
                    st_relaxed_u64(cx.pub + static_cast<size_t>(threadIdx.x) * cx.gmax + c,
                                   bound_word(e));
                __threadfence();
            }
        }
        take_bounds<Key, MIN>(st, cx, kth, publish);
        if (cnt > K) cnt = K;
    }
    TOPK_DUP(buf, cnt, mode == kFlushStream ? 4 : 2, done ? 0 : (cnt < K ? cnt : K), 3);
    // every thread has read st (nflush, ties, limit) for this flush's decisions before
    // thread 0 updates it (racecheck: without this barrier a late warp could read the
    // incremented nflush and take a different `done` -- a divergent CSync)
    CSync::sync();
    if (threadIdx.x == 0) {
        TOPK_STAT(0, 1ull);
        TOPK_STAT(1, static_cast<unsigned long long>(cnt0));
        TOPK_STAT(2, static_cast<unsigned long long>(clock64() - t0));
        if (!done) TOPK_STAT(6, 1ull);
        if (tried && !done && publish) st->ties = 1;
        {
            if (st->req & kReqBoot) {  // boot sample flushed (boot_sample): empty the bag
                for (int q = 0; q < st->nx; ++q) buf.st(q, st->xent[q]);  // (CTA 0)
                cnt = st->nx;
                done = true;
                bound_weaken1<Key, MIN>(st);  // keep >= the bound on re-read keys
            }
        }
        st->cnt = cnt;
        st->cnt_fail = 0x7FFFFFFF;
        st->sorted_cnt = done ? -1 : cnt;
        st->nflush += 1;
        st->limit = next_limit(st->nflush, K, cx.Lp, st->ties, cx.boot_l2);
        st->req = 0;
        trace(3);
    }
    CSync::sync();
}

// Collective bound refresh (no flush): rank bound over all CTAs' published samples.
template <class Key, bool MIN>
__device__ void refresh(CtaState<typename KeyTraits<Key>::E, Key>* st, const Ctx& cx) {
    using E = typename KeyTraits<Key>::E;
    load_pub(cx);
    CSync::sync();
    rank_rows(st, cx);
    if (threadIdx.x == 0) {
        TOPK_STAT(5, 1ull);
        fold_bounds<Key, MIN>(st, cx, E::sentinel());
        st->req = 0;
        trace(7);
    }
    CSync::sync();
}

// Boot sample (kBoot): each consumer thread appends the best entry among its keys of the
// first tile (positions as in consume_tile) and requests a flush, which the consumers
// run as their next collective (one flush call site: a second inlined copy of flush()
// spilled ~280 bytes per thread under the 128-register cap); that flush publishes the bag's
// samples and its k-th best (real entries of the input, so every bound derived from them
// is valid) and then empties the bag (kReqBoot) -- the tile is consumed next, against the
// boot bound weakened by one entry step: an entry EQUAL to the bound (its own k-th best,
// or its own sample coming back as the rank bound) was a bag entry and is now a new key
// again, and new keys must only be strictly better than the bound to be appended.
// Collective (consumers); the bag is empty on entry.
template <class Key, bool MIN>
__device__ void boot_sample(const unsigned char* slot_data, uint32_t tlen, uint32_t lbase,
                            const SBuf<typename KeyTraits<Key>::E>& buf,
                            CtaState<typename KeyTraits<Key>::E, Key>* st) {
    using KT = KeyTraits<Key>;
    using E = typename KT::E;
    constexpr int VEC = KT::kVec, ITEMS = Cfg<Key>::kItems;
    const Key* sk = reinterpret_cast<const Key*>(slot_data);
    const int tid = threadIdx.x;
    E m = E::sentinel();
#pragma unroll
    for (int q = 0; q < ITEMS; ++q) {
        const uint32_t pos = static_cast<uint32_t>((tid + (q / VEC) * kNC) * VEC + (q % VEC));
        if (pos < tlen) {
            const E e = E::make(KT::template code<MIN>(sk[pos]), lbase + pos);
            if (better(e, m)) m = e;
        }
    }
    const E ents[1] = {m};
    append<E, 1>(buf, &st->cnt, ents, m.is_sentinel() ? 0u : 1u, kCap);  // <= kNC entries
    CSync::sync();
    if (threadIdx.x == 0) st->req |= kReqFlush | kReqBoot;  // flushed by the collective
    CSync::sync();
}

// Consumer work on one tile held in shared memory.
//   fast pass: one compare per key against the threshold key, OR-reduced per warp --
//              the only work for the vast majority of tiles;
//   slow pass (some lane passed): per-key mask, exact entry test on the passing keys
//              (re-read from shared memory), warp prefix sum, one reservation, writes.
// Returns the buffer count before this warp's entries, or -1 if they did not fit.
template <class Key, bool MIN, bool FILTER>
__device__ __forceinline__ int consume_tile(const unsigned char* slot_data,
                                            const Par<typename KeyTraits<Key>::E, Key>& pr,
                                            uint32_t tlen, uint32_t lbase,
                                            const SBuf<typename KeyTraits<Key>::E>& buf,
                                            int* s_cnt, int limit) {
    using KT = KeyTraits<Key>;
    using E = typename KT::E;
    using Vec = typename KT::Vec;
    using C = Cfg<Key>;
    constexpr int VEC = KT::kVec;
    constexpr int VPT = C::kVecPerThread;
    constexpr int ITEMS = C::kItems;
    constexpr int TK = C::kTileKeys;
    const int tid = threadIdx.x;
    const int lane = tid & 31;

    const Vec* sv = reinterpret_cast<const Vec*>(slot_data);
    const Key* sk = reinterpret_cast<const Key*>(slot_data);
    Vec v[VPT];
#pragma unroll
    for (int j = 0; j < VPT; ++j) v[j] = sv[tid + j * kNC];

    const bool all = !FILTER || !pr.active;
    const bool strict = lbase > pr.strict_after;
    bool anyp = all;
    if (!all) {
        if (strict) {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                anyp |= KT::template fast<MIN, true>(vget(v[q / VEC], q % VEC), pr.t);
        } else {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                anyp |= KT::template fast<MIN, false>(vget(v[q / VEC], q % VEC), pr.t);
        }
    }
    if (!__any_sync(0xFFFFFFFFu, anyp)) return 0;

    uint32_t mask = 0;
    if (all) {
        mask = (ITEMS >= 32) ? 0xFFFFFFFFu : ((1u << ITEMS) - 1u);
    } else if (anyp) {
        if (strict) {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                mask |= static_cast<uint32_t>(
                            KT::template fast<MIN, true>(vget(v[q / VEC], q % VEC), pr.t)) << q;
        } else {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                mask |= static_cast<uint32_t>(
                            KT::template fast<MIN, false>(vget(v[q / VEC], q % VEC), pr.t)) << q;
        }
    }
    if (tlen < static_cast<uint32_t>(TK)) {
#pragma unroll
        for (int q = 0; q < ITEMS; ++q) {
            const uint32_t pos = static_cast<uint32_t>((tid + (q / VEC) * kNC) * VEC + q % VEC);
            if (pos >= tlen) mask &= ~(1u << q);
        }
    }
    auto pos_of = [&](int q) -> uint32_t {
        return static_cast<uint32_t>((tid + (q / VEC) * kNC) * VEC + (q % VEC));
    };
    uint32_t keep = mask;
    if (FILTER && pr.active) {  // exact entry test (R1 order) on the passing keys
        keep = 0;
        for (uint32_t m = mask; m; m &= m - 1u) {
            const int q = __ffs(m) - 1;
            const uint32_t pos = pos_of(q);
            const E e = E::make(KT::template code<MIN>(sk[pos]), lbase + pos);
            if (better(e, pr.tau)) keep |= 1u << q;
        }
    }
    const int cnt = __popc(keep);
    int incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    const int total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    if (total == 0) return 0;
    int old = 0;
    if (lane == 31) old = reserve(s_cnt, total, limit);
    old = __shfl_sync(0xFFFFFFFFu, old, 31);
    if (old < 0) return -1;
    int w = old + incl - cnt;
    for (uint32_t m = keep; m; m &= m - 1u) {
        const int q = __ffs(m) - 1;
        const uint32_t pos = pos_of(q);
        buf.st(w++, E::make(KT::template code<MIN>(sk[pos]), lbase + pos));
    }
    return old;
}

// Query form of consume_tile (Q != 0; filter mode): the row's key is the key column
// (or f = a + w * b), and a row enters the buffer filler only if it satisfies the
// predicate -- "apply the filter predicate ... and then [write] it out into a shared
// memory buffer" (FusedSortReducer), with the top-k bound as a second predicate.
// Keys stay in registers (<= 8 per thread) for the exact test.
template <class Key, bool MIN, int Q, bool SAMPLE = false>
__device__ __forceinline__ int consume_tile_q(const unsigned char* slot_data,
                                              const Par<typename KeyTraits<Key>::E, Key>& pr,
                                              uint32_t tlen, uint32_t lbase,
                                              const SBuf<typename KeyTraits<Key>::E>& buf,
                                              int* s_cnt, int limit, const SelectParams& p) {
    using KT = KeyTraits<Key>;
    using E = typename KT::E;
    using Vec = typename KT::Vec;
    using QC = QCfg<Key, Q>;
    constexpr int VEC = KT::kVec;
    constexpr int VPT = QC::kVecPerThread;
    constexpr int ITEMS = QC::kItems;
    constexpr int TK = QC::kTileKeys;
    // 4-byte secondary columns, VEC lanes at the key vector's positions
    using UVec = typename std::conditional<VEC == 4, uint4, uint2>::type;
    const int tid = threadIdx.x;
    const int lane = tid & 31;

    auto pos_of = [&](int q) -> uint32_t {
        return static_cast<uint32_t>((tid + (q / VEC) * kNC) * VEC + (q % VEC));
    };
    if constexpr ((Q & kQKey2) != 0) {
        // compound key: 64-bit codes (code(a) << 32 | code2(b)) [+ code3(c)].  The
        // streamed test is one float compare of the first key against the bound's first
        // key (non-strict: a superset of "may beat the bound"); only warps with a passing
        // row read the other columns and build codes for the exact entry test.
        float av[ITEMS];
        {
            const float4* sa = reinterpret_cast<const float4*>(slot_data);
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
                const float4 a = sa[tid + j * kNC];
#pragma unroll
                for (int w = 0; w < VEC; ++w) av[j * VEC + w] = vget(a, w);
            }
        }
        uint32_t mask = (ITEMS >= 32) ? 0xFFFFFFFFu : ((1u << ITEMS) - 1u);
        if (tlen < static_cast<uint32_t>(TK)) {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                if (pos_of(q) >= tlen) mask &= ~(1u << q);
        }
        if (pr.active) {
            const float t1 = KeyTraits<float>::template decode<MIN>(pr.tau.c >> 32);
            uint32_t f = 0;
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                f |= static_cast<uint32_t>(KeyTraits<float>::template fast<MIN, false>(av[q], t1)) << q;
            mask &= f;
            if (!__any_sync(0xFFFFFFFFu, mask != 0u)) return 0;
        }
        if constexpr ((Q & kQPred) != 0) {
            const uint4* sp = reinterpret_cast<const uint4*>(slot_data + QC::kOffP);
            uint32_t pm = 0;
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
                const uint4 u = sp[tid + j * kNC];
#pragma unroll
                for (int w = 0; w < VEC; ++w)
                    pm |= static_cast<uint32_t>(pred_ok(p, vget(u, w))) << (j * VEC + w);
            }
            mask &= pm;
        }
        uint64_t cc[ITEMS];
        uint32_t c3[ITEMS];
        {
            const float4* sb = reinterpret_cast<const float4*>(slot_data + QC::kOffB);
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
                const float4 b = sb[tid + j * kNC];
#pragma unroll
                for (int w = 0; w < VEC; ++w)
                    cc[j * VEC + w] = KT::template code2<MIN>(av[j * VEC + w], vget(b, w), p.order2_min);
            }
        }
        if constexpr ((Q & kQKey3) != 0) {
            const float4* sc = reinterpret_cast<const float4*>(slot_data + QC::kOffC);
#pragma unroll
            for (int j = 0; j < VPT; ++j) {
                const float4 cv = sc[tid + j * kNC];
#pragma unroll
                for (int w = 0; w < VEC; ++w) c3[j * VEC + w] = KT::code3(vget(cv, w), p.order3_min);
            }
        }
        auto mk = [&](int q) -> E {
            if constexpr ((Q & kQKey3) != 0)
                return E::make(cc[q], c3[q], lbase + pos_of(q));
            else
                return E::make(cc[q], lbase + pos_of(q));
        };
        if (pr.active) {  // exact entry test (lexicographic codes, then the row)
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                if (((mask >> q) & 1u) && !better(mk(q), pr.tau)) mask &= ~(1u << q);
        }
        if constexpr (SAMPLE) {  // boot sample: the thread's best matching row only
            E m = E::sentinel();
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                if (((mask >> q) & 1u) && better(mk(q), m)) m = mk(q);
            const E one[1] = {m};
            return append<E, 1>(buf, s_cnt, one, m.is_sentinel() ? 0u : 1u, limit);
        }
        E ents[ITEMS];
#pragma unroll
        for (int q = 0; q < ITEMS; ++q) ents[q] = mk(q);
        return append<E, ITEMS>(buf, s_cnt, ents, mask, limit);
    } else {
    Key x[ITEMS];
    {
        const Vec* sv = reinterpret_cast<const Vec*>(slot_data);
#pragma unroll
        for (int j = 0; j < VPT; ++j) {
            const Vec v = sv[tid + j * kNC];
#pragma unroll
            for (int w = 0; w < VEC; ++w) x[j * VEC + w] = vget(v, w);
        }
    }
    if constexpr ((Q & kQRank) != 0) {
        static_assert(sizeof(Key) == 4 && VEC == 4, "ranking function: f32 columns");
        const float4* sb = reinterpret_cast<const float4*>(slot_data + QC::kOffB);
#pragma unroll
        for (int j = 0; j < VPT; ++j) {
            const float4 b = sb[tid + j * kNC];
#pragma unroll
            for (int w = 0; w < VEC; ++w) x[j * VEC + w] = rank_f(x[j * VEC + w], p.rank_w, vget(b, w));
        }
    }
    uint32_t pm = (ITEMS >= 32) ? 0xFFFFFFFFu : ((1u << ITEMS) - 1u);
    if constexpr ((Q & kQPred) != 0) {
        const UVec* sp = reinterpret_cast<const UVec*>(slot_data + QC::kOffP);
        pm = 0;
#pragma unroll
        for (int j = 0; j < VPT; ++j) {
            const UVec u = sp[tid + j * kNC];
#pragma unroll
            for (int w = 0; w < VEC; ++w)
                pm |= static_cast<uint32_t>(pred_ok(p, vget(u, w))) << (j * VEC + w);
        }
    }
    if (tlen < static_cast<uint32_t>(TK)) {
#pragma unroll
        for (int q = 0; q < ITEMS; ++q)
            if (pos_of(q) >= tlen) pm &= ~(1u << q);
    }
    uint32_t mask = pm;
    if (pr.active) {
        const bool strict = lbase > pr.strict_after;
        uint32_t f = 0;
        if (strict) {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                f |= static_cast<uint32_t>(KT::template fast<MIN, true>(x[q], pr.t)) << q;
        } else {
#pragma unroll
            for (int q = 0; q < ITEMS; ++q)
                f |= static_cast<uint32_t>(KT::template fast<MIN, false>(x[q], pr.t)) << q;
        }
        mask &= f;
    }
    if (!__any_sync(0xFFFFFFFFu, mask != 0u)) return 0;
    uint32_t keep = mask;
    if (pr.active) {  // exact entry test (R1 order) on the passing rows
        keep = 0;
#pragma unroll
        for (int q = 0; q < ITEMS; ++q)
            if (((mask >> q) & 1u) &&
                better(E::make(KT::template code<MIN>(x[q]), lbase + pos_of(q)), pr.tau))
                keep |= 1u << q;
    }
    if constexpr (SAMPLE) {  // boot sample: the thread's best matching row only
        E m = E::sentinel();
#pragma unroll
        for (int q = 0; q < ITEMS; ++q) {
            const E e = E::make(KT::template code<MIN>(x[q]), lbase + pos_of(q));
            if (((keep >> q) & 1u) && better(e, m)) m = e;
        }
        const E one[1] = {m};
        return append<E, 1>(buf, s_cnt, one, m.is_sentinel() ? 0u : 1u, limit);
    }
    const int cnt = __popc(keep);
    int incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    const int total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    if (total == 0) return 0;
    int old = 0;
    if (lane == 31) old = reserve(s_cnt, total, limit);
    old = __shfl_sync(0xFFFFFFFFu, old, 31);
    if (old < 0) return -1;
    int w = old + incl - cnt;
#pragma unroll
    for (int q = 0; q < ITEMS; ++q)
        if ((keep >> q) & 1u) buf.st(w++, E::make(KT::template code<MIN>(x[q]), lbase + pos_of(q)));
    return old;
    }
}

// The key of global row `row` under query form Q (the extras and the finalize gather).
template <class Key, int Q>
__device__ __forceinline__ Key query_key(const SelectParams& p, const Key* keys, uint64_t row) {
    if constexpr ((Q & kQRank) != 0)
        return rank_f(keys[row], p.rank_w, p.col_b[row]);
    else
        return keys[row];
}
// The entry of global row `row` (< 2^32 - 1) under query form Q.
template <class Key, bool MIN, int Q>
__device__ __forceinline__ typename KeyTraits<Key>::E query_entry(const SelectParams& p,
                                                                  const Key* keys, uint64_t row) {
    using KT = KeyTraits<Key>;
    if constexpr ((Q & kQKey3) != 0)
        return KT::E::make(KT::template code2<MIN>(keys[row].a, p.col_b[row], p.order2_min),
                           KT::code3(p.col_c[row], p.order3_min), static_cast<uint32_t>(row));
    else if constexpr ((Q & kQKey2) != 0)
        return KT::E::make(KT::template code2<MIN>(keys[row].a, p.col_b[row], p.order2_min),
                           static_cast<uint32_t>(row));
    else
        return KT::E::make(KT::template code<MIN>(query_key<Key, Q>(p, keys, row)),
                           static_cast<uint32_t>(row));
}


// Tail: append ITEMS entries per thread (mask = which) to the bag, flushing (final mode)
// whenever a warp's entries do not fit.  Collective over the consumer warps.
template <class Key, bool MIN, int ITEMS>
__device__ __forceinline__ void append_all(const SBuf<typename KeyTraits<Key>::E>& buf,
                                           CtaState<typename KeyTraits<Key>::E, Key>* st,
                                           const Ctx& cx,
                                           const typename KeyTraits<Key>::E (&ents)[ITEMS],
                                           uint32_t mask) {
    using E = typename KeyTraits<Key>::E;
    bool todo = true;
    while (true) {
        int vote = 0;
        if (todo) {
            if (__any_sync(0xFFFFFFFFu, mask != 0u)) {
                const int old = append<E, ITEMS>(buf, &st->cnt, ents, mask, kCap);
                todo = old < 0;
                vote = todo ? 1 : 0;
            } else {
                todo = false;
            }
        }
        if (!cbar_or(vote != 0)) break;
        flush<Key, MIN>(buf, st, cx, kFlushFinal);
    }
}

template <class Key, bool MIN, bool FILTER, int Q = 0>
__global__ void __launch_bounds__(kNT, 1) select_kernel(const SelectParams p) {
    using KT = KeyTraits<Key>;
    using E = typename KT::E;
    using C = Cfg<Key>;
    constexpr int TK = QCfg<Key, Q>::kTileKeys;
    using QC = QCfg<Key, Q>;
    constexpr int kStages = QC::kStages;
    constexpr int kSlot = QC::kSlotBytes;
    static_assert(Q == 0 || FILTER, "query forms run in filter mode");
    // Boot sample (plain form, f32 / u32 / f64 keys): the boot bag is the best key of each
    // consumer thread's share of the first tile (480 entries, each the best of 16 -- f64: 8
    // -- keys) instead of
    // the tile's first keys -- the same flush, a 16x larger sample behind its bound.  The
    // bag is then emptied and the tile consumed as usual.
    constexpr bool kBoot = FILTER && TOPK_BOOT_SAMPLE && (Q == 0 || TOPK_BOOT_SAMPLE_Q) &&
                           (!std::is_same<E, E96>::value || TOPK_BOOT_SAMPLE_E96);

    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ CtaState<E, Key> st;

    unsigned char* ring = smem;
    SBuf<E> buf;
    buf.init(smem + static_cast<size_t>(kStages) * kSlot, kCap);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + static_cast<size_t>(kStages) * kSlot +
                                                 static_cast<size_t>(kCap) * SBuf<E>::kBytes);
    uint64_t* empty = full + kStages;
    unsigned long long* scratch = reinterpret_cast<unsigned long long*>(empty + kStages);

    const int tid = threadIdx.x;
    const uint32_t G = gridDim.x;
    const uint32_t c = blockIdx.x;
    const int K = static_cast<int>(p.K);
    const int k = static_cast<int>(p.k);
    // Before the first flush every key is kept: the boot buffer is the boot sample
    // (st.limit = kCap); after it, next_limit().
    const Key* keys = static_cast<const Key*>(p.keys);
    WsHeader* hdr = reinterpret_cast<WsHeader*>(p.ws);
    Ctx cx;
    uint32_t refresh_at;  // tile index at which consumer thread 0 requests a rank-bound refresh
    cx.hdr = hdr;
    cx.pub = reinterpret_cast<unsigned long long*>(p.ws + ws_pub_offset());
    cx.scratch = scratch;
    cx.k = k;
    cx.K = K;
    cx.G = static_cast<int>(G);
    cx.gmax = static_cast<int>(p.gmax);
    cx.J = static_cast<int>(p.J);
    cx.j_lo = 0;
    while (cx.j_lo < cx.J && ((k + (1 << cx.j_lo) - 1) >> cx.j_lo) > cx.G) ++cx.j_lo;
    {
        const int maxrows = (c_dbg >> 4) & 3 ? (c_dbg >> 4) & 3 : 3;
        cx.nrows = cx.J - cx.j_lo < maxrows ? cx.J - cx.j_lo : maxrows;
    }
    cx.filter = FILTER;
    // Second flush after a boot sample (measured, 2^29 uniform): K <= 256 -- none (the
    // boot bound is tight enough; k = 128 348 -> 338 us, k = 256 354 -> 352); larger K
    // (the 480-entry boot bag has no k-th best) -- as soon as the bag holds 4x the
    // deepest sample the stream rank bound uses (k = 1024: 64 entries, 391 -> 373 us;
    // k = 2048: 128)
    // Boot wait (measured with the boot sample): K <= 256 proceed on their own boot bound and
    // pull the rank bound at tile 6 (k = 32 331 -> 328 us, k = 256 354 -> 352); larger K wait
    // (without it k = 1024 375 -> 399 us) and refresh at tile 12
    cx.boot_wait = !kBoot || K >= TOPK_BOOT_WAIT_KMIN;
    refresh_at = cx.boot_wait ? TOPK_REFRESH_AT : TOPK_REFRESH_AT_NOWAIT;
    cx.boot_l2 = !kBoot ? 0
                 : K <= TOPK_L2_BOOT_KMAX ? kCap
                 : TOPK_L2_BOOT_MUL << (cx.j_lo + min(cx.nrows, TOPK_FLUSH_ROWS) - 1);
    // K > 512: the code network still gives the bag's 2^j-th best codes for j <= 9,
    // whose cross-CTA rank bound bounds the global k-th best (t = ceil(k / 2^j) <= G)
    cx.Lp = FILTER ? (K < 16 ? 4 : min(__ffs(K) - 1, 9)) : -1;
    cx.codes = scratch + kScratch;

    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kNC / 32);
        }
        fence_mbar_init();
        st.cnt = 0;
        st.nx = 0;
        st.perm_mode = 0;
        st.cnt_fail = 0x7FFFFFFF;
        st.req = 0;
        st.nflush = 0;
        st.sorted_cnt = -1;
        st.pubd = 0;
        // boot buffer: every CTA flushes it at about the same time (the HBM idles), so
        // large K -- whose flush costs more -- boots on a small sample (measured with the
        // c_dbg knob, 2^29 uniform f32: K >= 256 best with 512 entries -- k = 256 379 ->
        // 363 us, k = 1024 406 -> 396 us; K <= 128 best with the whole buffer)
        st.limit = (c_dbg >> 8) & 7 ? kCap >> ((c_dbg >> 8) & 7)
                   : (K >= TOPK_BOOT_SMALL_K && !kBoot) ? kCap / 8 : kCap;
        st.ties = 0;
        st.tau_w = 0ull;
        st.tau = E::sentinel();
        st.par = make_par<Key, MIN>(E::sentinel());
    }
    // Extras: the unaligned head and the sub-16-byte tail, appended by CTA 0 to an empty
    // bag (at the start, or after the boot sample's flush).
    auto append_extras = [&]() {
        const uint64_t tail0 = p.head + p.body_n;
        const int nextra = static_cast<int>(p.head + (p.n - tail0));
        if constexpr (Q == 0) {
            if (tid < nextra) {
                const uint64_t row = tid < static_cast<int>(p.head) ? static_cast<uint64_t>(tid)
                                                                     : tail0 + (tid - p.head);
                buf.st(tid, E::make(KT::template code<MIN>(keys[row]), static_cast<uint32_t>(row)));
            }
            if (tid == 0) st.cnt = nextra;
        } else if (tid < 32) {  // query forms: head == 0, nextra <= 3; WHERE applies
            const uint64_t row = tail0 + tid;
            bool ok = tid < nextra;
            if constexpr ((Q & kQPred) != 0) ok = ok && pred_ok(p, p.pred[ok ? row : 0]);
            const uint32_t bal = __ballot_sync(0xFFFFFFFFu, ok);
            if (ok) buf.st(__popc(bal & ((1u << tid) - 1u)), query_entry<Key, MIN, Q>(p, keys, row));
            if (tid == 0) st.cnt = __popc(bal);
        }
    };
    if (c == 0) {
        if constexpr (kBoot) {  // kept aside: the boot flush empties the bag, then adds them
            const uint64_t tail0 = p.head + p.body_n;
            const int nextra = static_cast<int>(p.head + (p.n - tail0));
            if constexpr (Q == 0) {
                if (tid < nextra) {
                    const uint64_t row = tid < static_cast<int>(p.head) ? static_cast<uint64_t>(tid)
                                                                         : tail0 + (tid - p.head);
                    st.xent[tid] = E::make(KT::template code<MIN>(keys[row]), static_cast<uint32_t>(row));
                }
                if (tid == 0) st.nx = nextra;
            } else if (tid < 32) {  // query forms: head == 0, nextra <= 3; WHERE applies
                const uint64_t row = tail0 + tid;
                bool ok = tid < nextra;
                if constexpr ((Q & kQPred) != 0) ok = ok && pred_ok(p, p.pred[ok ? row : 0]);
                const uint32_t bal = __ballot_sync(0xFFFFFFFFu, ok);
                if (ok) st.xent[__popc(bal & ((1u << tid) - 1u))] = query_entry<Key, MIN, Q>(p, keys, row);
                if (tid == 0) st.nx = __popc(bal);
            }
        } else {
            append_extras();
        }
    }
    __syncthreads();

    // Wave order (TOPK_ADAPTIVE_ORDER): waves after the first are visited in a pseudo-random
    // order only if the input looks sorted -- 64 probe keys spread over it, >= 90 % of
    // their neighbour pairs strictly increasing or strictly decreasing (every CTA probes
    // the same keys, so every CTA takes the same decision).  A sorted input read in
    // address order keeps raising the bound (every new wave beats all earlier ones: 2^29
    // increasing, k = 256: 1064 us); any other input streams faster in address order
    // (uniform 352 -> 345 us, few-distinct 369 -> 332, decreasing 360 -> 325).
    if (tid < 32) {
        const int lane0 = tid;
        int mode = p.perm_h > 0 ? 2 : 1;
        if constexpr (FILTER && Q == 0 && TOPK_ADAPTIVE_ORDER) {
            if (p.perm_h > 0 && p.n >= 128) {
                const uint64_t stp = p.n / 64;
                const auto c0 = KT::template code<MIN>(keys[static_cast<uint64_t>(2 * lane0) * stp]);
                const auto c1 = KT::template code<MIN>(keys[static_cast<uint64_t>(2 * lane0 + 1) * stp]);
                const auto nx = __shfl_down_sync(0xFFFFFFFFu, c0, 1);
                // signs of the 63 neighbour differences (probe j -> j + 1): d0 = c1 - c0,
                // d1 = next lane's c0 - c1
                const int s0 = c1 > c0 ? 1 : (c1 < c0 ? -1 : 0);
                const int s1 = lane0 < 31 ? (nx > c1 ? 1 : (nx < c1 ? -1 : 0)) : 0;
                const int sn = __shfl_down_sync(0xFFFFFFFFu, s0, 1);  // next lane's d0
                int inc = (s0 > 0) + (s1 > 0), dec = (s0 < 0) + (s1 < 0);
                // neighbouring differences of one sign: ~1/3 of the 62 for i.i.d. keys,
                // nearly all for piecewise monotone input
                int agree = (s0 != 0 && s0 == s1) + (lane0 < 31 && s1 != 0 && s1 == sn);
                inc = __reduce_add_sync(0xFFFFFFFFu, inc);
                dec = __reduce_add_sync(0xFFFFFFFFu, dec);
                agree = __reduce_add_sync(0xFFFFFFFFu, agree);
                // ascending codes (the best keys at the end): the waves backwards; descending
                // codes (the best keys first): forwards; other piecewise monotone input (organ
                // pipe, sawtooth): permuted; anything else: forwards
                mode = inc >= 57 ? 3 : dec >= 57 ? 1 : agree >= 50 ? 2 : 1;
            }
        }
        if (lane0 == 0) *reinterpret_cast<volatile int*>(&st.perm_mode) = mode;
    }

    if (tid >= kNC) {
        // ---------------- producer warp (lane 0) ----------------
        if (tid != kNC) return;
        const Key* body = keys + p.head;
        const uint64_t policy = l2_evict_first_policy();
        const uint32_t blk = p.blk;
        const uint32_t nclaim = p.nwaves * p.wave * blk;
        uint32_t claim = 0, left = 0;
        int mode = 0;  // wave order (st.perm_mode), read once
        uint32_t pending = atomicAdd(&hdr->next_tile, blk);
#pragma unroll 1
        for (uint32_t s = 0;; ++s) {
            const int slot = static_cast<int>(s % kStages);
            uint32_t tile = kEndTile;
            while (true) {
                if (left == 0) {
                    claim = pending;  // consumes the outstanding claim
                    left = blk;
                    if (claim >= nclaim) break;
                    pending = atomicAdd(&hdr->next_tile, blk);
                }
                const uint32_t i = claim++;
                --left;
                // claim i -> block b = (wave, position); waves permuted, the blocks of a
                // wave adjacent; tiles of a block in address order
                const uint32_t b = i / blk;
                // address order, or the waves permuted (decided by the probe, which
                // lands while the first claim's atomic is in flight)
                const uint32_t wv = b / p.wave;
                uint32_t pw = wv;
                if (p.perm_h) {
                    while (mode == 0) mode = *reinterpret_cast<volatile int*>(&st.perm_mode);
                    if (mode == 2) pw = feistel_perm(wv, p.nwaves, p.perm_h);
                    if (mode == 3) pw = p.nwaves - 1u - wv;
                }
                const uint32_t pb = pw * p.wave + b % p.wave;
                const uint32_t t = pb * blk + i % blk;
                if (t < p.ntiles) {
                    tile = t;
                    break;
                }
            }
            if (s >= static_cast<uint32_t>(kStages))
                mbar_wait(&empty[slot], ((s / kStages) - 1u) & 1u);
            st.tile[slot] = tile;
            if (tile == kEndTile) {
                mbar_arrive(&full[slot]);  // no bytes: the consumers see kEndTile
                return;
            }
            const uint64_t lo = static_cast<uint64_t>(tile) * TK;
            const uint64_t len = min(static_cast<uint64_t>(TK), p.body_n - lo);
            uint32_t bytes = static_cast<uint32_t>(len * sizeof(Key));
            unsigned char* dst = ring + static_cast<size_t>(slot) * kSlot;
            tma_load_1d(dst, body + lo, bytes, &full[slot], policy);
            if constexpr ((Q & (kQRank | kQKey2)) != 0) {  // one slab per column (head == 0)
                tma_load_1d(dst + QCfg<Key, Q>::kOffB, p.col_b + lo,
                            static_cast<uint32_t>(len * 4), &full[slot], policy);
                bytes += static_cast<uint32_t>(len * 4);
            }
            if constexpr ((Q & kQKey3) != 0) {
                tma_load_1d(dst + QCfg<Key, Q>::kOffC, p.col_c + lo, static_cast<uint32_t>(len * 4),
                            &full[slot], policy);
                bytes += static_cast<uint32_t>(len * 4);
            }
            if constexpr ((Q & kQPred) != 0) {
                tma_load_1d(dst + QCfg<Key, Q>::kOffP, p.pred + lo, static_cast<uint32_t>(len * 4),
                            &full[slot], policy);
                bytes += static_cast<uint32_t>(len * 4);
            }
            mbar_arrive_expect_tx(&full[slot], bytes);  // release: tile id visible
        }
    }

    // ---------------- consumer warps ----------------
    const int lane = tid & 31;
    if (tid == 0) trace(1);
    auto pending_req = [&]() -> bool { return *reinterpret_cast<volatile int*>(&st.req) != 0; };
    // Body of a collective, entered by all consumer warps after one OR-barrier.
    auto collective = [&]() {
        if (st.req & kReqFlush)
            flush<Key, MIN>(buf, &st, cx, kFlushStream);
        else
            refresh<Key, MIN>(&st, cx);
    };
    uint32_t ntiles_done = 0;
    if constexpr (kBoot) {
        // boot sample: wait for the first slot, append each thread's best key of it and
        // request its flush -- the main loop's first wait runs that flush as a collective
        // and then consumes the same tile.  (A CTA without tiles appends the extras here;
        // otherwise the boot flush does, after emptying the bag.)
        while (!__all_sync(0xFFFFFFFFu, mbar_try_wait(&full[0], 0u))) {
        }
        uint32_t tile = 0;
        if (lane == 0) tile = st.tile[0];
        tile = __shfl_sync(0xFFFFFFFFu, tile, 0);
        if (tile != kEndTile) {
            const uint32_t tlen = static_cast<uint32_t>(
                min(static_cast<uint64_t>(TK), p.body_n - static_cast<uint64_t>(tile) * TK));
            const uint32_t lbase = static_cast<uint32_t>(p.head + static_cast<uint64_t>(tile) * TK);
            if constexpr (Q == 0) {
                boot_sample<Key, MIN>(ring, tlen, lbase, buf, &st);
            } else {  // the thread's best row passing the WHERE, same entry as consume_tile_q
                consume_tile_q<Key, MIN, Q, true>(ring, make_par<Key, MIN>(E::sentinel()), tlen,
                                                  lbase, buf, &st.cnt, kCap, p);
                CSync::sync();
                if (tid == 0) st.req |= kReqFlush | kReqBoot;  // flushed by the collective
                CSync::sync();
            }
        } else {
            if (tid == 0) {
                for (int q = 0; q < st.nx; ++q) buf.st(q, st.xent[q]);
                st.cnt = st.nx;
            }
            CSync::sync();
        }
    }
#pragma unroll 1
    for (uint32_t s = 0;; ++s) {
        const int slot = static_cast<int>(s % kStages);
        const uint32_t parity = (s / kStages) & 1u;
        // warp-uniform wait (synccheck): a lane must not enter a collective while another
        // lane of its warp is still polling the ring
        while (true) {
            if (__any_sync(0xFFFFFFFFu, pending_req())) {
                cbar_or(true);
                collective();
                continue;
            }
            if (__all_sync(0xFFFFFFFFu, mbar_try_wait(&full[slot], parity))) break;
        }
        // (lane 0 -- the lane that arrives on empty[slot] -- reads the tile id: every
        // read of st.tile[slot] is then ordered before the producer's next write of it by
        // that arrive, which racecheck can see)
        uint32_t tile = 0;
        if (lane == 0) tile = st.tile[slot];
        tile = __shfl_sync(0xFFFFFFFFu, tile, 0);
        if (tile == kEndTile) break;
        ++ntiles_done;
#ifdef TOPK_DUPCHECK
        if (tid == 0 && tile < (1u << 16)) atomicAdd(&g_tiles[tile], 1u);
#endif
        const uint64_t tlo = static_cast<uint64_t>(tile) * TK;
        const uint32_t tlen = static_cast<uint32_t>(min(static_cast<uint64_t>(TK), p.body_n - tlo));
        const uint32_t lbase = static_cast<uint32_t>(p.head + tlo);
        const unsigned char* data = ring + static_cast<size_t>(slot) * kSlot;
        Par<E, Key> pr = load_par<Key, MIN>(st);
        auto consume = [&]() -> int {
            if constexpr (Q == 0)
                return consume_tile<Key, MIN, FILTER>(data, pr, tlen, lbase, buf, &st.cnt, st.limit);
            else
                return consume_tile_q<Key, MIN, Q>(data, pr, tlen, lbase, buf, &st.cnt, st.limit, p);
        };
        int r = consume();
        while (r < 0) {  // did not fit: flush, then redo with the new bound
            if (lane == 0) {
                TOPK_STAT(3, 1ull);
                atomicOr(&st.req, kReqFlush);
            }
            __syncwarp();
            cbar_or(true);
            collective();
            pr = load_par<Key, MIN>(st);
            r = consume();
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[slot]);
        // Once every CTA has had time to publish its first run, pull the rank bound.
        if (FILTER && G > 1 && tid == 0 && s == refresh_at) atomicOr(&st.req, kReqRefresh);
    }
    // Drain: serve requests of warps still streaming, until all are done.
    while (cbar_or(pending_req())) collective();
    if (tid == 0) trace(4);
    if (tid == 0) {
        TOPK_STAT(4, static_cast<unsigned long long>(ntiles_done));
        if (!st.pubd) atomicAdd(&hdr->npub, 1u);  // peers waiting at boot need not wait for us
    }
    // The CTA's run: the exact top-K of its bag, best first (skipped if already sorted).
    if (st.cnt == 0) {
        for (int j = tid; j < K; j += kNC) buf.st(j, E::sentinel());
        CSync::sync();
    } else if (st.cnt != st.sorted_cnt) {
        TOPK_DUP(buf, st.cnt, 1, 0, 3);
        flush<Key, MIN>(buf, &st, cx, kFlushFinal);
    }

    // ---- hand the CTA's top-k to the reduction (last CTA to arrive) ----
    GBuf<E> cand;
    cand.init(p.ws + ws_cand_offset(p.gmax), static_cast<size_t>(G) * k);
    if (tid == 0) st.cnt_run = st.cnt;
    if (G > 1) {
        for (int j = tid; j < k; j += kNC) cand.st(static_cast<size_t>(c) * k + j, buf.ld(j));
        __threadfence();
        CSync::sync();
        if (tid == 0) st.last = (atomicAdd(&hdr->ticket, 1u) == G - 1u) ? 1 : 0;
        CSync::sync();
        if (!st.last) return;
        __threadfence();
        if (tid == 0) trace(5);
        const unsigned long long tau_g_w =
            tid == 0 ? ld_relaxed_u64(reinterpret_cast<const uint64_t*>(&hdr->tau_g)) : 0ull;
        // (1) Stage the first kk entries of every other run in the idle ring (one L2 round
        // trip for all of them; every run is sorted best first, so only a prefix of it can
        // reach the global top-k).
        if (cx.nrows > TOPK_TAIL_ROWS) cx.nrows = TOPK_TAIL_ROWS;
        constexpr int kEB = SBuf<E>::kBytes;
        int kk = 1;
        while (kk * 2 <= k && kk < 32) kk *= 2;  // largest power of two <= min(k, 32)
        const int deep = 1 << (cx.j_lo + cx.nrows - 1);  // deepest rank-bound sample + 1
        while (kk < deep && kk * 2 <= k) kk *= 2;
        while (kk > 1 && ((static_cast<int>(G) * kk + 15) & ~15) * kEB > kStages * kSlot) kk >>= 1;
        const int lk = __ffs(kk) - 1;
        const int nst = static_cast<int>(G) << lk;
        SBuf<E> stg;
        stg.init(ring, (nst + 15) & ~15);
        {
            constexpr int U = 4;  // loads in flight per thread
            for (int q0 = tid; q0 < nst; q0 += U * kNC) {
                E v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int q = q0 + u * kNC;
                    const int cc = q >> lk;
                    v[u] = (q < nst && cc != static_cast<int>(c))
                               ? cand.ld(static_cast<size_t>(cc) * k + (q & (kk - 1)))
                               : E::sentinel();
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (q0 + u * kNC < nst) stg.st(q0 + u * kNC, v[u]);
            }
        }
        CSync::sync();
        // (2) Rank bound over the final runs (tail form of the flush bound): row j holds
        // each run's 2^j-th best (from the staged prefixes where they lie inside them);
        // the t-th largest (t = ceil(k / 2^j) <= G) bounds the global k-th best.
        {
            const int S = scr_stride(cx.G);
            for (int q = tid; q < cx.nrows * S; q += kNC) {
                const int ji = cx.j_lo + q / S, cc = q % S;
                const int pos = (1 << ji) - 1;
                const E e = cc >= cx.G ? E::sentinel()
                            : (pos < kk && cc != static_cast<int>(c))
                                ? stg.ld((cc << lk) + pos)
                                : cand.ld(static_cast<size_t>(cc) * k + pos);
                scratch[q] = bound_word(e);
            }
        }
        CSync::sync();
        if (tid == 0) trace(8);
        rank_rows(&st, cx);
        if (tid == 0) trace(9);
        if (tid == 0) {
            E tb = from_bound_word<E>(tau_g_w);
            for (int ji = 0; ji < kPubRows; ++ji) {
                const E b = from_bound_word<E>(st.best[ji]);
                if (st.best[ji] != 0ull && better(b, tb)) tb = b;
            }
            if (st.cnt_run >= k && better(buf.ld(k - 1), tb)) tb = buf.ld(k - 1);
            st.tau = tb;
            st.cnt = 0;
            st.req = 0;
        }
        CSync::sync();
        const E tb = st.tau;
        {   // own run: keep its qualifying prefix (sorted best first)
            const int own = st.cnt_run < k ? st.cnt_run : k;
            int q = 0;
            for (int j = tid; j < own; j += kNC) q += better(tb, buf.ld(j)) ? 0 : 1;
            q = __reduce_add_sync(0xFFFFFFFFu, q);
            if (lane == 0 && q) atomicAdd(&st.cnt, q);
            CSync::sync();
            if (tid == 0) st.sorted_cnt = st.cnt;
            CSync::sync();
        }
        if (tid == 0) trace(11);
        // (3) Append the qualifying staged entries; flag the runs whose last staged entry
        // still qualified (their tails kk .. k are appended in (4)).
        __shared__ unsigned int s_more[(kGMax + 31) / 32];
        __shared__ int s_flag_list[kGMax];
        __shared__ int s_nflag;
        for (int q = tid; q < (kGMax + 31) / 32; q += kNC) s_more[q] = 0u;
        CSync::sync();
        constexpr int CI = 11;
        for (int q0 = 0; q0 < nst; q0 += CI * kNC) {
            E ents[CI];
            uint32_t mask = 0;
#pragma unroll
            for (int r = 0; r < CI; ++r) {
                const int q = q0 + tid + r * kNC;
                ents[r] = q < nst ? stg.ld(q) : E::sentinel();
                if (!ents[r].is_sentinel() && !better(tb, ents[r])) {
                    mask |= 1u << r;
                    if ((q & (kk - 1)) == kk - 1 && kk < k) {
                        const int cc = q >> lk;
                        atomicOr(&s_more[cc >> 5], 1u << (cc & 31));
                    }
                }
            }
            if (tid == 0) trace(25);
            append_all<Key, MIN, CI>(buf, &st, cx, ents, mask);
            if (tid == 0) trace(26);
        }
        CSync::sync();
        if (tid == 0) trace(12);
        // (4) The rest (positions kk .. k) of the flagged runs (rare: a run with more than
        // kk entries in the global top-k).
        if (kk < k) {
            if (tid < 32) {  // warp 0: ballot-based compaction of the flag bits
                int nf = 0;
                for (int w0 = 0; w0 < (cx.G + 31) / 32; ++w0) {
                    const int cc = w0 * 32 + tid;
                    const bool f = cc < cx.G && ((s_more[w0] >> tid) & 1u);
                    const uint32_t bal = __ballot_sync(0xFFFFFFFFu, f);
                    if (f) s_flag_list[nf + __popc(bal & ((1u << tid) - 1u))] = cc;
                    nf += __popc(bal);
                }
                if (tid == 0) s_nflag = nf;
            }
            CSync::sync();
            const int span = k - kk;
            const int lsp = 32 - __clz(span - 1 > 0 ? span - 1 : 0);  // next_pow2(span)
            const int total = s_nflag << lsp;
            for (int q0 = 0; q0 < total; q0 += CI * kNC) {
                E ents[CI];
                uint32_t mask = 0;
                size_t at[CI];
                bool ok[CI];
#pragma unroll
                for (int r = 0; r < CI; ++r) {
                    const int q = q0 + tid + r * kNC;
                    const int j = q & ((1 << lsp) - 1);
                    ok[r] = q < total && j < span;
                    at[r] = ok[r] ? static_cast<size_t>(s_flag_list[q >> lsp]) * k + kk + j : 0;
                }
#pragma unroll
                for (int r = 0; r < CI; ++r) ents[r] = cand.ld(at[r]);
#pragma unroll
                for (int r = 0; r < CI; ++r) {
                    if (ok[r] && !ents[r].is_sentinel() && !better(tb, ents[r]))
                        mask |= 1u << r;
                    else
                        ents[r] = E::sentinel();
                }
                append_all<Key, MIN, CI>(buf, &st, cx, ents, mask);
            }
            CSync::sync();
        }
        if (tid == 0) trace(10);
        if (tid == 0) trace(32 + min(st.cnt >> 6, 31));
        TOPK_DUP(buf, st.cnt, 5, 0, 3);
        if (st.cnt != st.sorted_cnt) flush<Key, MIN>(buf, &st, cx, kFlushFinal);
        TOPK_DUP(buf, k, 6, k, 3);
    }
    // ---- finalize: best first, original key bits, global index, payload ----
    for (int j = tid; j < k; j += kNC) {
        const E e = buf.ld(j);
        if (e.is_sentinel()) {  // fewer than k rows (only a WHERE can do that, since k <= n)
            if (Q == 0) TOPK_STAT(7, 1ull);  // plain form: a bug
            if (p.out_idx) p.out_idx[j] = -1;
            if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = Key{0};
            if constexpr ((Q & kQKey2) != 0)
                if (p.out_keys2) p.out_keys2[j] = 0.f;
            if constexpr ((Q & kQKey3) != 0)
                if (p.out_keys3) p.out_keys3[j] = 0.f;
            if (p.out_payload) p.out_payload[j] = 0u;
            continue;
        }
        const uint32_t row = e.lidx();
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(p.base + row);
        if constexpr ((Q & kQKey2) != 0) {
            if (p.out_keys) static_cast<float*>(p.out_keys)[j] = keys[row].a;
            if (p.out_keys2) p.out_keys2[j] = p.col_b[row];
            if constexpr ((Q & kQKey3) != 0)
                if (p.out_keys3) p.out_keys3[j] = p.col_c[row];
        } else {
            if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = query_key<Key, Q>(p, keys, row);
        }
        if (p.out_payload) p.out_payload[j] = p.payload[row];
    }
    if (tid == 0) trace(6);
#ifdef TOPK_DUPCHECK
    for (uint32_t q = tid; q < p.ntiles && q < (1u << 16); q += kNC) {
        const unsigned int v = g_tiles[q];
        if (v != 1u) atomicAdd(&g_stats[v == 0u ? 0 : 7], 1ull);
        g_tiles[q] = 0u;
    }
#endif
    // leave the workspace zeroed for the next call (all other CTAs are done)
    for (int q = tid; q < kPubRows * static_cast<int>(G); q += kNC)
        cx.pub[static_cast<size_t>(q / G) * p.gmax + q % G] = 0ull;
    if (tid == 0) {
        hdr->tau_g = 0ull;
        hdr->ticket = 0u;
        hdr->npub = 0u;
        hdr->next_tile = 0u;
    }
}

template <class Key, int Q = 0>
constexpr size_t select_smem_bytes() {
    return static_cast<size_t>(QCfg<Key, Q>::kStages) * QCfg<Key, Q>::kSlotBytes +
           static_cast<size_t>(kCap) * SBuf<typename KeyTraits<Key>::E>::kBytes +
           static_cast<size_t>(2 * QCfg<Key, Q>::kStages) * 8 + static_cast<size_t>(kScratch) * 8 +
           static_cast<size_t>(kCap / 512) * 512 *
               sizeof(typename CodeOf<typename KeyTraits<Key>::E>::C);  // code network
}

}  // namespace topk
