// radix.cuh -- radix-select top-k, the paper's selection-based alternative (§2.3 "Radix
// Select"; §4.2 "Selection-based Top-K"; cost model §7.1),
// built B200-native so the bench can put the two methods side by side.
//
// MSD radix select over the order code (keys.cuh; larger = better), 8-bit digits "based
// on MSD radix sort ... 4 passes for 32 bit keys", 8 passes for 64-bit codes:
//   digit pass j: histogram of digit j over the current candidates (the input filtered
//     by the known prefix, or the bucket) -> prefix sum from the top -> the digit d_j
//     of the bucket holding the k-th best code ("uses the histogram to find the bucket
//     B containing the k-th-largest entry");
//   "writes out only the entries of B" -- here the bucket is written
//     once (scatter), after the first digit whose bucket fits the workspace; before
//     that "the clustering step is skipped and we simply re-use the input in the next
//     pass" -- U(0,1) floats put half the keys in one first-digit bucket;
//   "when scanning the array the second time to write out the tuples that fall into
//     the bucket, we can also write out the elements in the higher buckets to a
//     separate result array" -- the scatter pass appends every entry above
//     the bucket to the result candidates.
// After the last digit the k-th best code X is known exactly.  The result is every
// entry with code > X plus the lowest-index entries with code == X (the tie rule of
// DESIGN.md R1 -- the paper pads "with X", which fixes values but not rows):
// collected from the bucket (collect pass) or, when the bucket path was skipped or the
// ties are too many, from one more input pass that keeps, per CTA slice in row order,
// the first ties ("one additional pass over the input array").  A final CTA
// sorts the k entries best first with the local sort / merge / rebuild network
// (network.cuh) and gathers the original key bits.
//
// Every decision is taken on the device (state in the workspace): the launch sequence
// is fixed, kernels whose work was made unnecessary exit at once, no host sync.
#pragma once
#include "cnet.cuh"  // CodeOf
#include "keys.cuh"
#include "merge.cuh"
#include "network.cuh"

namespace topk {

constexpr int kRadixNT = 256;                  // threads per CTA of the scans
constexpr int kRadixPerThread = 16;            // keys per thread per tile
constexpr int kRadixTile = kRadixNT * kRadixPerThread;
constexpr int kRadixEqCap = 4096;              // ties collected from the bucket
constexpr int kRadixBins = 256;                // 8-bit digits

template <class C>
struct RadixEntry {
    C code;
    uint32_t lidx;
};

template <class C>
struct RadixState {
    C prefix;            // known top digits of X (bits above `shift`)
    uint32_t shift;      // bit position of the next digit
    uint32_t k_rem;      // rank of X inside the current candidates (1-based)
    uint32_t bucket_ok;  // 1: a bucket was written (later passes read it)
    uint32_t nbucket;    // entries written to the bucket
    uint32_t ngt;        // result candidates with code > X (exactly k - m at the end)
    uint32_t neq;        // ties (code == X) collected from the bucket
    uint32_t need_emit;  // 1: the final input pass collects gt / ties
    uint32_t scatter;    // 1: the bucket of the digit just chosen is written next
    uint32_t bshift;     // bit position of the digit just chosen
    uint32_t pad;
};

struct RadixParams {
    const void* keys;
    uint64_t n;
    uint64_t base;
    uint32_t k, K;
    uint32_t G;          // CTAs of the input passes (contiguous slices)
    uint64_t slice;      // keys per CTA slice (multiple of kRadixTile)
    uint32_t cap;        // bucket capacity (entries)
    unsigned char* ws;
    void* out_keys;
    int64_t* out_idx;
};

// Workspace layout: [state | hist 256 (+ spare) | gt k | eq kRadixEqCap | eqc G x k |
// eqn G | bucket cap].
template <class C>
struct RadixWs {
    RadixState<C>* st;
    uint32_t* hist;  // [256] digit totals of the current pass
    RadixEntry<C>* gt;
    RadixEntry<C>* eq;
    RadixEntry<C>* eqc;
    uint32_t* eqn;
    RadixEntry<C>* bucket;
};
__host__ __device__ inline size_t radix_align(size_t x) { return (x + 255) / 256 * 256; }
template <class C>
__host__ __device__ inline size_t radix_ws_bytes(uint32_t G, uint32_t k, uint32_t cap) {
    const size_t e = sizeof(RadixEntry<C>);
    return radix_align(sizeof(RadixState<C>)) + radix_align(size_t(G) * kRadixBins * 4) +
           radix_align(k * e) + radix_align(kRadixEqCap * e) + radix_align(size_t(G) * k * e) +
           radix_align(size_t(G) * 4) + radix_align(size_t(cap) * e);
}
template <class C>
__host__ __device__ inline RadixWs<C> radix_ws(unsigned char* ws, uint32_t G, uint32_t k) {
    const size_t e = sizeof(RadixEntry<C>);
    RadixWs<C> w;
    size_t o = 0;
    w.st = reinterpret_cast<RadixState<C>*>(ws + o);
    o += radix_align(sizeof(RadixState<C>));
    w.hist = reinterpret_cast<uint32_t*>(ws + o);
    o += radix_align(size_t(G) * kRadixBins * 4);
    w.gt = reinterpret_cast<RadixEntry<C>*>(ws + o);
    o += radix_align(k * e);
    w.eq = reinterpret_cast<RadixEntry<C>*>(ws + o);
    o += radix_align(kRadixEqCap * e);
    w.eqc = reinterpret_cast<RadixEntry<C>*>(ws + o);
    o += radix_align(size_t(G) * k * e);
    w.eqn = reinterpret_cast<uint32_t*>(ws + o);
    o += radix_align(size_t(G) * 4);
    w.bucket = reinterpret_cast<RadixEntry<C>*>(ws + o);
    return w;
}

template <class C>
__device__ __forceinline__ uint32_t digit_of(C c, uint32_t shift) {
    return static_cast<uint32_t>(c >> shift) & 0xFFu;
}
// Does code c carry the known prefix (the bits above `shift`)?
template <class C>
__device__ __forceinline__ bool has_prefix(C c, C prefix, uint32_t shift) {
    constexpr uint32_t kBits = sizeof(C) * 8;
    return shift + 8 >= kBits ? true : (c >> (shift + 8)) == (prefix >> (shift + 8));
}

// The keys of one tile of a CTA slice: thread t owns 16 consecutive keys (row order
// = thread order, so a block scan gives row-ordered offsets).
template <class Key, bool MIN>
__device__ __forceinline__ int load_codes(const Key* keys, uint64_t n, uint64_t row0,
                                          typename CodeOf<typename KeyTraits<Key>::E>::C (&c)[kRadixPerThread]) {
    using KT = KeyTraits<Key>;
    using Vec = typename KT::Vec;
    constexpr int VEC = KT::kVec;
    if (row0 + kRadixPerThread <= n && (reinterpret_cast<uintptr_t>(keys + row0) & 15) == 0) {
        const Vec* v = reinterpret_cast<const Vec*>(keys + row0);  // 128-bit loads
#pragma unroll
        for (int j = 0; j < kRadixPerThread / VEC; ++j) {
            const Vec x = __ldg(v + j);
            if constexpr (VEC == 4) {
                c[4 * j] = KT::template code<MIN>(x.x);
                c[4 * j + 1] = KT::template code<MIN>(x.y);
                c[4 * j + 2] = KT::template code<MIN>(x.z);
                c[4 * j + 3] = KT::template code<MIN>(x.w);
            } else {
                c[2 * j] = KT::template code<MIN>(x.x);
                c[2 * j + 1] = KT::template code<MIN>(x.y);
            }
        }
        return kRadixPerThread;
    }
    int valid = 0;
#pragma unroll
    for (int q = 0; q < kRadixPerThread; ++q) {
        const uint64_t r = row0 + q;
        if (r < n) {
            c[q] = KT::template code<MIN>(__ldg(keys + r));
            ++valid;
        } else {
            c[q] = 0;
        }
    }
    return valid;
}

// Block-wide exclusive scan of one count per thread (kRadixNT threads).
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* s_w, uint32_t* total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += y;
    }
    __syncthreads();
    if (lane == 31) s_w[w] = incl;
    __syncthreads();
    uint32_t off = 0, all = 0;
#pragma unroll
    for (int i = 0; i < kRadixNT / 32; ++i) {
        const uint32_t x = s_w[i];
        off += i < w ? x : 0;
        all += x;
    }
    *total = all;
    return off + incl - v;
}

// Warp-aggregated append of `take` entries to list[*cnt ...] (one atomic per warp).
template <class C>
__device__ __forceinline__ void warp_append(RadixEntry<C>* list, uint32_t* cnt, uint32_t cap,
                                            bool take, RadixEntry<C> e, uint32_t* overflow) {
    const int lane = threadIdx.x & 31;
    const uint32_t m = __ballot_sync(0xFFFFFFFFu, take);
    if (!m) return;
    uint32_t base = 0;
    const int leader = __ffs(m) - 1;
    if (lane == leader) base = atomicAdd(cnt, static_cast<uint32_t>(__popc(m)));
    base = __shfl_sync(0xFFFFFFFFu, base, leader);
    const uint32_t pos = base + __popc(m & ((1u << lane) - 1u));
    if (take) {
        if (pos < cap) list[pos] = e;
        else if (overflow) *overflow = 1u;
    }
}

// Digit pass: per-CTA histogram of digit `shift` over the candidates -- the input
// filtered by the known prefix (pass 1, or while no bucket was written), else the
// bucket.  Counts only; the choice is made by radix_choose.  One 256-bin histogram
// per warp in shared memory, fire-and-forget shared atomics (no result is waited for,
// so a thread's 16 increments pipeline; same-bin lanes serialise in the atomic unit --
// U(0,1) floats put half the keys on one first digit), warps summed at the end.
#ifndef TOPK_RADIX_MATCH
#define TOPK_RADIX_MATCH 0
#endif
constexpr int kHistNT = 256;
// kHistCopies histograms per warp (lane % kHistCopies), rows padded by one word so the
// copies of one bin sit in different banks: U(0,1) floats put half the keys on one first
// digit, and same-address shared atomics of a warp serialise
#ifndef TOPK_HIST_COPIES
#define TOPK_HIST_COPIES 1
#endif
constexpr int kHistCopies = TOPK_HIST_COPIES;
constexpr int kHistRow = kRadixBins + 1;
template <class Key, bool MIN, bool FIRST>
__global__ void __launch_bounds__(kHistNT) radix_hist(const RadixParams p) {
    using C = typename CodeOf<typename KeyTraits<Key>::E>::C;
    constexpr int kRows = kHistNT / 32 * kHistCopies;
    __shared__ uint32_t hw[kRows][kHistRow];
    const int warp = threadIdx.x >> 5;
    const RadixWs<C> w = radix_ws<C>(p.ws, p.G, p.k);
    for (int i = threadIdx.x; i < kRows * kHistRow; i += kHistNT) (&hw[0][0])[i] = 0u;
    uint32_t* mine = hw[warp * kHistCopies + (threadIdx.x & 31) % kHistCopies];
    const C prefix = FIRST ? C(0) : w.st->prefix;
    const uint32_t shift = FIRST ? sizeof(C) * 8 - 8 : w.st->shift;
    const bool from_bucket = !FIRST && w.st->bucket_ok;
    __syncthreads();
    if (from_bucket) {
        const uint32_t nb = w.st->nbucket;
        for (uint32_t i = blockIdx.x * kHistNT + threadIdx.x; i < nb; i += gridDim.x * kHistNT) {
            const C c = w.bucket[i].code;
            if (has_prefix(c, prefix, shift)) atomicAdd(&mine[digit_of(c, shift)], 1u);
        }
    } else {
        const Key* keys = static_cast<const Key*>(p.keys);
        const uint64_t lo = blockIdx.x * p.slice, hi = min(p.n, lo + p.slice);
        constexpr int kT = kHistNT * kRadixPerThread;
        // two tiles in flight per thread (the loads of the next tile are issued before the
        // counts of the current one: the pass is bound by memory-level parallelism)
        C cn[kRadixPerThread];
        load_codes<Key, MIN>(keys, hi, lo + threadIdx.x * kRadixPerThread, cn);
        for (uint64_t t0 = lo; t0 < hi; t0 += kT) {
            C c[kRadixPerThread];
#pragma unroll
            for (int q = 0; q < kRadixPerThread; ++q) c[q] = cn[q];
            const uint64_t r0 = t0 + threadIdx.x * kRadixPerThread;
            if (t0 + kT < hi) load_codes<Key, MIN>(keys, hi, r0 + kT, cn);
#pragma unroll
            for (int q = 0; q < kRadixPerThread; ++q) {
                const bool ok = r0 + q < hi && has_prefix(c[q], prefix, shift);
#if TOPK_RADIX_MATCH
                // lanes with the same digit add once (U(0,1) floats put half the keys on
                // one first digit: same-address shared atomics would serialise)
                const uint32_t d = ok ? digit_of(c[q], shift) : 0x100u + (threadIdx.x & 31);
                const uint32_t peers = __match_any_sync(0xFFFFFFFFu, d);
                if (ok && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&mine[d], __popc(peers));
#else
                if (ok) atomicAdd(&mine[digit_of(c[q], shift)], 1u);
#endif
            }
        }
    }
    __syncthreads();
    for (int b = threadIdx.x; b < kRadixBins; b += kHistNT) {
        uint32_t s = 0;
#pragma unroll
        for (int wv = 0; wv < kRows; ++wv) s += hw[wv][b];
        if (s) atomicAdd(&w.hist[b], s);  // the pass's total (radix_choose reads and zeroes it)
    }
}

// Prefix sum from the top digit down: the bucket d holding the k_rem-th best code
// (P:93).  One CTA of 256 threads (one per digit value).  FIRST also initialises the
// state and decides whether the bucket is written (it fits the workspace).
template <class C, bool FIRST>
__global__ void __launch_bounds__(kRadixBins) radix_choose(const RadixParams p) {
    __shared__ uint32_t tot[kRadixBins];
    __shared__ uint32_t s_w[kRadixBins / 32];
    const RadixWs<C> w = radix_ws<C>(p.ws, p.G, p.k);
    RadixState<C>* st = w.st;
    const int d = threadIdx.x;
    uint32_t s = 0;
    s = w.hist[d];
    w.hist[d] = 0u;  // ready for the next digit pass
    tot[d] = s;
    __syncthreads();
    if (d == 0) {
        if (FIRST) {
            st->prefix = 0;
            st->shift = sizeof(C) * 8 - 8;
            st->k_rem = p.k;
            st->nbucket = 0;
            st->ngt = 0;
            st->neq = 0;
            st->need_emit = 0;
            st->bucket_ok = 0;
        }
        st->scatter = 0;
    }
    __syncthreads();
    // above[d] = sum of tot over digits > d: inclusive scan from the top
    const uint32_t v = tot[kRadixBins - 1 - d];
    uint32_t total;
    const uint32_t excl = block_excl_scan(v, s_w, &total);
    const uint32_t above = excl;  // entries with a digit > (255 - d)
    const uint32_t kr = st->k_rem;
    __syncthreads();
    const int dig = kRadixBins - 1 - d;
    if (above < kr && kr <= above + v) {  // exactly one digit satisfies this
        const uint32_t shift = st->shift;
        st->prefix = st->prefix | (static_cast<C>(dig) << shift);
        st->k_rem = kr - above;
        // write the bucket once, as soon as it fits the workspace ("if after the prefix
        // sum we see no data reduction, the clustering step is skipped")
        if (!st->bucket_ok && v <= p.cap) {
            st->scatter = 1;
            st->bucket_ok = 1;
        }
        st->bshift = shift;
        st->shift = shift >= 8 ? shift - 8 : 0;
        if (shift == 0) st->shift = 0xFFFFFFFFu;  // done: prefix == X
    }
}

// After the digit whose bucket first fits the workspace: write the bucket (entries
// whose code carries the prefix chosen so far) and append every entry above it to the
// result.  Exits at once at the other digits.
template <class Key, bool MIN>
__global__ void __launch_bounds__(kRadixNT) radix_scatter(const RadixParams p) {
    using C = typename CodeOf<typename KeyTraits<Key>::E>::C;
    const RadixWs<C> w = radix_ws<C>(p.ws, p.G, p.k);
    if (!w.st->scatter) return;
    const uint32_t kTop = w.st->bshift;
    const C d1 = w.st->prefix >> kTop;
    // bucket entries are staged per warp in shared memory (warp-aggregated appends, no
    // CTA barrier) and written with one global reservation per warp flush
    constexpr int kWStage = 256;
    __shared__ RadixEntry<C> stage[kRadixNT / 32][kWStage];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t lt = (1u << lane) - 1u;
    uint32_t staged = 0;  // warp-uniform
    auto wflush = [&]() {
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(&w.st->nbucket, staged);
        base = __shfl_sync(0xFFFFFFFFu, base, 0);
        for (uint32_t i = lane; i < staged; i += 32)
            if (base + i < p.cap) w.bucket[base + i] = stage[warp][i];
        __syncwarp();
        staged = 0;
    };
    const Key* keys = static_cast<const Key*>(p.keys);
    const uint64_t lo = blockIdx.x * p.slice, hi = min(p.n, lo + p.slice);
    for (uint64_t t0 = lo; t0 < hi; t0 += kRadixTile) {
        C c[kRadixPerThread];
        const uint64_t r0 = t0 + threadIdx.x * kRadixPerThread;
        load_codes<Key, MIN>(keys, hi, r0, c);
        uint32_t gtm = 0;
#pragma unroll
        for (int q = 0; q < kRadixPerThread; ++q) {
            const bool ok = r0 + q < hi;
            const C dg = c[q] >> kTop;  // code above the bucket's bits
            gtm |= static_cast<uint32_t>(ok && dg > d1) << q;
            const bool in = ok && dg == d1;
            const uint32_t m = __ballot_sync(0xFFFFFFFFu, in);
            if (m) {
                if (staged + __popc(m) > kWStage) wflush();
                if (in) stage[warp][staged + __popc(m & lt)] =
                            RadixEntry<C>{c[q], static_cast<uint32_t>(r0 + q)};
                staged += __popc(m);
            }
        }
        // entries above the bucket: fewer than k in all (rare: one vote per tile, then
        // warp-aggregated appends)
        if (__any_sync(0xFFFFFFFFu, gtm != 0u)) {
#pragma unroll
            for (int q = 0; q < kRadixPerThread; ++q)
                warp_append(w.gt, &w.st->ngt, p.k, (gtm >> q) & 1u,
                            RadixEntry<C>{c[q], static_cast<uint32_t>(r0 + q)}, nullptr);
        }
    }
    __syncwarp();
    if (staged) wflush();
}

// After the last digit (prefix == X): from the bucket, entries with code > X join the
// result, ties (code == X) are collected (up to kRadixEqCap; more -> the input pass).
template <class C>
__global__ void __launch_bounds__(kRadixNT) radix_collect(const RadixParams p) {
    const RadixWs<C> w = radix_ws<C>(p.ws, p.G, p.k);
    RadixState<C>* st = w.st;
    if (!st->bucket_ok) {
        if (blockIdx.x == 0 && threadIdx.x == 0) st->need_emit = 1;
        return;
    }
    const C X = st->prefix;
    const uint32_t nb = st->nbucket;
    const uint32_t n_iter = (nb + gridDim.x * kRadixNT - 1) / (gridDim.x * kRadixNT);
    for (uint32_t it = 0; it < n_iter; ++it) {
        const uint32_t i = (it * gridDim.x + blockIdx.x) * kRadixNT + threadIdx.x;
        RadixEntry<C> e{C(0), 0u};
        if (i < nb) e = w.bucket[i];
        warp_append(w.gt, &st->ngt, p.k, i < nb && e.code > X, e, nullptr);
        warp_append(w.eq, &st->neq, kRadixEqCap, i < nb && e.code == X, e, &st->need_emit);
    }
}

// The additional input pass, needed when the bucket was not written or the
// ties overflowed: per CTA slice, in row order, entries with code > X join the result
// and the first k ties are kept in eqc[cta] (row order within the slice).
template <class Key, bool MIN>
__global__ void __launch_bounds__(kRadixNT) radix_emit(const RadixParams p) {
    using C = typename CodeOf<typename KeyTraits<Key>::E>::C;
    __shared__ uint32_t s_w[kRadixNT / 32];
    const RadixWs<C> w = radix_ws<C>(p.ws, p.G, p.k);
    RadixState<C>* st = w.st;
    if (!st->need_emit) return;
    // with the bucket written, scatter + collect already found every code > X (only the
    // ties overflowed); otherwise this pass finds them
    const bool add_gt = !st->bucket_ok;
    const C X = st->prefix;
    const Key* keys = static_cast<const Key*>(p.keys);
    const uint64_t lo = blockIdx.x * p.slice, hi = min(p.n, lo + p.slice);
    uint32_t taken = 0;  // ties kept by this CTA so far
    RadixEntry<C>* mine = w.eqc + static_cast<size_t>(blockIdx.x) * p.k;
    for (uint64_t t0 = lo; t0 < hi; t0 += kRadixTile) {
        C c[kRadixPerThread];
        const uint64_t r0 = t0 + threadIdx.x * kRadixPerThread;
        load_codes<Key, MIN>(keys, hi, r0, c);
        uint32_t ne = 0;
#pragma unroll
        for (int q = 0; q < kRadixPerThread; ++q) {
            const bool ok = r0 + q < hi;
            ne += (ok && c[q] == X) ? 1u : 0u;
            if (add_gt)
                warp_append(w.gt, &st->ngt, p.k, ok && c[q] > X,
                            RadixEntry<C>{c[q], static_cast<uint32_t>(r0 + q)}, nullptr);
        }
        uint32_t tile_eq;
        uint32_t pos = taken + block_excl_scan(ne, s_w, &tile_eq);
        if (taken < p.k && ne) {
#pragma unroll
            for (int q = 0; q < kRadixPerThread; ++q)
                if (r0 + q < hi && c[q] == X) {
                    if (pos < p.k) mine[pos] = RadixEntry<C>{c[q], static_cast<uint32_t>(r0 + q)};
                    ++pos;
                }
        }
        taken += tile_eq;
    }
    if (threadIdx.x == 0) w.eqn[blockIdx.x] = taken < p.k ? taken : p.k;
}

// Final CTA: the k result entries (every code > X, then the lowest-row ties), sorted
// best first by the paper's network (local sort / merge / rebuild, network.cuh) on
// (code, global row) entries; original key bits gathered by row.  Leaves the state
// zeroed for the next call.
template <class Key, bool MIN>
__global__ void __launch_bounds__(kMergeNT, 1) radix_final(const RadixParams p) {
    using C = typename CodeOf<typename KeyTraits<Key>::E>::C;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ uint32_t s_take[2];
    SBuf<EM> buf;
    buf.init(smem, kMergeCap);
    const RadixWs<C> w = radix_ws<C>(p.ws, p.G, p.k);
    RadixState<C>* st = w.st;
    const int tid = threadIdx.x;
    const int K = static_cast<int>(p.K), k = static_cast<int>(p.k);
    const uint32_t ngt = min(st->ngt, p.k);
    auto ent = [&](const RadixEntry<C>& e) {
        return EM{static_cast<uint64_t>(e.code), p.base + e.lidx, e.lidx};
    };
    for (uint32_t i = tid; i < ngt; i += kMergeNT) buf.st(i, ent(w.gt[i]));
    int cnt = static_cast<int>(ngt);
    if (!st->need_emit) {
        // ties from the bucket (unordered): all of them; the network keeps the lowest rows
        const uint32_t neq = min(st->neq, static_cast<uint32_t>(kRadixEqCap));
        for (uint32_t i = tid; i < neq; i += kMergeNT) buf.st(cnt + i, ent(w.eq[i]));
        cnt += static_cast<int>(neq);
    } else {
        // ties from the input pass: slices in row order, the first k - ngt of them
        if (tid == 0) {
            uint32_t need = p.k - ngt, at = 0;
            for (uint32_t c = 0; c < p.G && need; ++c) {
                const uint32_t t = min(w.eqn[c], need);
                for (uint32_t j = 0; j < t; ++j)
                    buf.st(cnt + static_cast<int>(at + j), ent(w.eqc[static_cast<size_t>(c) * p.k + j]));
                at += t;
                need -= t;
            }
            s_take[0] = at;
        }
        __syncthreads();
        cnt += static_cast<int>(s_take[0]);
    }
    int P = 2 * K;
    while (P < cnt) P <<= 1;
    for (int i = cnt + tid; i < P; i += kMergeNT) buf.st(i, EM::sentinel());
    __syncthreads();
    bitonic_topk_smem<EM, kMergeNT, CtaSync>(buf, P, K);
    const Key* keys = static_cast<const Key*>(p.keys);
    for (int j = tid; j < k; j += kMergeNT) {
        const EM e = buf.ld(j);
        if (p.out_idx) p.out_idx[j] = static_cast<int64_t>(e.idx);
        if (p.out_keys) static_cast<Key*>(p.out_keys)[j] = keys[e.row];
    }
    __syncthreads();
    if (tid == 0) {  // zero the state for the next call
        st->ngt = 0;
        st->neq = 0;
        st->nbucket = 0;
        st->need_emit = 0;
        st->bucket_ok = 0;
        st->scatter = 0;
    }
}

}  // namespace topk
