// topk_api.cu -- the C ABI declared in include/topk.h: argument validation, planning
// (alignment peel, tiles, grid, tile permutation), workspace layout, and dispatch of
// the sm_100a kernels.  No host synchronisation, no allocation.
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "merge.cuh"
#include "probe.cuh"
#include "dispatch.h"
#include "pure.cuh"
#include "radix.cuh"
#include "select.cuh"
#include "topk.h"

namespace {

std::atomic<uint64_t> g_launches{0};

struct DevInfo {
    int sms = 0;
    int major = 0;
    bool ok = false;
};
DevInfo g_dev[64];

bool device_info(int* sms, int* major) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return false;
    DevInfo& d = g_dev[dev];
    if (!d.ok) {
        if (cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
            return false;
        if (cudaDeviceGetAttribute(&d.major, cudaDevAttrComputeCapabilityMajor, dev) !=
            cudaSuccess)
            return false;
        d.ok = true;
    }
    *sms = d.sms;
    *major = d.major;
    return true;
}

size_t key_size(topk_dtype_t dt) { return dt == TOPK_F64 ? 8 : 4; }
// workspace candidate entry bytes: 8 (32-bit codes); 12 for f64 / two compound keys,
// 16 for three compound keys (E96) -- the 64-bit layouts share the larger size
size_t entry_bytes(topk_dtype_t dt) { return dt == TOPK_F64 ? 16 : 8; }

uint32_t next_pow2_u32(uint32_t x) {
    uint32_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

bool valid_dtype(int dt) { return dt == TOPK_F32 || dt == TOPK_U32 || dt == TOPK_F64; }
bool valid_order(int o) { return o == TOPK_LARGEST || o == TOPK_SMALLEST; }

// Largest n one launch indexes with a 32-bit local row id (0xFFFFFFFF is reserved for
// the sentinel entry).
constexpr uint64_t kMaxLaunchN = 0xFFFFFFFEull;

// One select kernel instantiation per generated TU (dispatch.h kSelectTable).
cudaError_t launch_variant(int key, bool min_order, bool filter, int q,
                           const topk::SelectParams& p, int grid, cudaStream_t st) {
    for (int i = 0; i < topk::kSelectTableN; ++i) {
        const topk::SelectEntry& v = topk::kSelectTable[i];
        if (v.key == key && v.min == (min_order ? 1 : 0) && v.filter == (filter ? 1 : 0) &&
            v.q == q) {
            const cudaError_t e = v.launch(p, grid, st);
            if (e == cudaSuccess) g_launches.fetch_add(1, std::memory_order_relaxed);
            return e;
        }
    }
    return cudaErrorInvalidValue;  // no such instantiation
}

int key_kind(topk_dtype_t dt) {
    return dt == TOPK_F64 ? topk::kKeyF64 : dt == TOPK_U32 ? topk::kKeyU32 : topk::kKeyF32;
}

template <class Key, bool MIN>
cudaError_t launch_merge(const topk::MergeParams& p, cudaStream_t st) {
    static std::atomic<uint64_t> attr_set{0};  // per device (dispatch.h)
    const cudaError_t e = topk::smem_attr_once(topk::merge_kernel<Key, MIN>,
                                               static_cast<int>(topk::kMergeSmem), attr_set);
    if (e != cudaSuccess) return e;
    topk::merge_kernel<Key, MIN><<<1, topk::kMergeNT, topk::kMergeSmem, st>>>(p);
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return cudaGetLastError();
}

template <class Key>
cudaError_t dispatch_merge(const topk::MergeParams& p, bool min_order, cudaStream_t st) {
    return min_order ? launch_merge<Key, true>(p, st) : launch_merge<Key, false>(p, st);
}

template <class Key>
uint32_t tile_keys() {
    return static_cast<uint32_t>(topk::Cfg<Key>::kTileKeys);
}

uint32_t tile_keys_for(topk_dtype_t dt) {
    switch (dt) {
        case TOPK_F64: return tile_keys<double>();
        case TOPK_U32: return tile_keys<uint32_t>();
        default: return tile_keys<float>();
    }
}

uint32_t query_tile_keys(topk_dtype_t dt, int q) {
    using topk::QCfg;
    using topk::kQPred;
    using topk::kQRank;
    using topk::kQKey2;
    using topk::kQKey3;
    if (q & kQKey3)
        return (q & kQPred) ? QCfg<topk::KKK32, kQKey2 | kQKey3 | kQPred>::kTileKeys
                            : QCfg<topk::KKK32, kQKey2 | kQKey3>::kTileKeys;
    if (q & kQKey2)
        return (q & kQPred) ? QCfg<topk::KK32, kQKey2 | kQPred>::kTileKeys
                            : QCfg<topk::KK32, kQKey2>::kTileKeys;
    if (dt == TOPK_F64) return QCfg<double, kQPred>::kTileKeys;
    if (dt == TOPK_U32) return QCfg<uint32_t, kQPred>::kTileKeys;
    switch (q) {
        case kQRank: return QCfg<float, kQRank>::kTileKeys;
        case kQRank | kQPred: return QCfg<float, kQRank | kQPred>::kTileKeys;
        default: return QCfg<float, kQPred>::kTileKeys;
    }
}

// Candidate area: one run of next_pow2(k) entries per CTA (the pure-mode kernel keeps
// whole K-runs; the streaming select keeps k).
size_t select_ws_bytes(topk_dtype_t dtype, uint32_t k, int sms) {
    const size_t runs = static_cast<size_t>(sms) + (sms + topk::kPureGroup - 1) / topk::kPureGroup;
    return align_up(topk::ws_cand_offset(static_cast<uint32_t>(sms)) +
                        runs * next_pow2_u32(k) * entry_bytes(dtype),
                    256);
}

}  // namespace

// Merge `total` candidate entries (contiguous) to the exact top-k (topk_merge's body).
// run_len: entries per run (the last run may be shorter); sorted: every run is sorted
// best first (topk_select's output), so the merge kernel skips the local sort.
static topk_status_t merge_total(topk_dtype_t dtype, const void* cand_keys,
                                 const int64_t* cand_idx, const uint32_t* cand_payload,
                                 uint64_t total, uint32_t run_len, bool sorted, uint32_t k,
                                 topk_order_t order, void* out_keys, uint32_t* out_payload,
                                 int64_t* out_idx, void* stream, bool ordered = false,
                                 const uint64_t* ranges = nullptr);
// chunked-input helpers (used by topk_workspace_bytes / topk_select).  Chunk length
// 2^31 keys; TOPK_CHUNK_N (multiple of 4) overrides it so tests can exercise the
// chunked path on small inputs.
static uint64_t chunk_n() {
    static const uint64_t v = [] {
        const char* e = std::getenv("TOPK_CHUNK_N");
        const unsigned long long x = e ? std::strtoull(e, nullptr, 10) : 0ull;
        return (x >= 4096 && x % 4 == 0 && x <= (1ull << 31)) ? static_cast<uint64_t>(x)
                                                              : (1ull << 31);
    }();
    return v;
}
struct ChunkLayout {
    size_t sel, ck, ci, cp, total;  // offsets of: select ws, cand keys, ids, payloads
};
static ChunkLayout chunk_layout(topk_dtype_t dtype, uint64_t nchunks, uint32_t k, int sms) {
    ChunkLayout L;
    L.sel = 0;
    L.ck = align_up(select_ws_bytes(dtype, k, sms), 256);
    L.ci = L.ck + align_up(nchunks * k * key_size(dtype), 256);
    L.cp = L.ci + align_up(nchunks * k * 8, 256);
    L.total = L.cp + align_up(nchunks * k * 4, 256);
    return L;
}

extern "C" {

size_t topk_workspace_bytes(topk_dtype_t dtype, uint64_t n, uint32_t k) {
    if (!valid_dtype(dtype) || n == 0 || k == 0 || k > TOPK_MAX_K || k > n) return 0;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return 0;
    if (n <= kMaxLaunchN && n <= chunk_n()) return select_ws_bytes(dtype, k, sms);
    const uint64_t nch = (n + chunk_n() - 1) / chunk_n();
    return chunk_layout(dtype, nch, k, sms).total;
}

topk_status_t topk_workspace_init(void* ws, size_t ws_bytes, void* stream) {
    if (!ws || ws_bytes < sizeof(topk::WsHeader)) return TOPK_ERR_WORKSPACE;
    if (cudaMemsetAsync(ws, 0, ws_bytes, static_cast<cudaStream_t>(stream)) != cudaSuccess)
        return TOPK_ERR_CUDA;
    return TOPK_OK;
}

// Query forms (topk_query): q = kQPred | kQRank bits, 0 for a plain top-k.
struct QueryArgs {
    int q = 0;
    const float* rank_b = nullptr;
    float rank_w = 0.f;
    topk_pred_t pred{};
    float* out_keys2 = nullptr;  // kQKey2
    uint32_t order2_min = 0;
    const float* col_c = nullptr;  // kQKey3
    float* out_keys3 = nullptr;
    uint32_t order3_min = 0;
};

static topk_status_t select_one(topk_dtype_t dtype, const void* keys, const uint32_t* payload,
                          uint64_t n, uint64_t base, uint32_t k, topk_order_t order,
                          topk_mode_t mode, void* out_keys, uint32_t* out_payload,
                          int64_t* out_idx, void* ws, size_t ws_bytes, void* stream,
                          const QueryArgs& qa = QueryArgs()) {
    if (!valid_dtype(dtype) || !valid_order(order)) return TOPK_ERR_INVALID_ARG;
    if (mode != TOPK_MODE_FILTER && mode != TOPK_MODE_PURE) return TOPK_ERR_INVALID_ARG;
    if (!keys || n == 0 || k == 0 || k > TOPK_MAX_K || k > n) return TOPK_ERR_INVALID_ARG;
    if (out_payload && !payload) return TOPK_ERR_INVALID_ARG;
    const size_t ks = key_size(dtype);
    const uintptr_t addr = reinterpret_cast<uintptr_t>(keys);
    if (addr % ks) return TOPK_ERR_INVALID_ARG;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return TOPK_ERR_CUDA;
    if (major != 10 || sms > topk::kGMax) return TOPK_ERR_UNSUPPORTED;
    const size_t need = select_ws_bytes(dtype, k, sms);
    if (!ws || ws_bytes < need || (reinterpret_cast<uintptr_t>(ws) % 256)) return TOPK_ERR_WORKSPACE;

    topk::SelectParams p;
    std::memset(&p, 0, sizeof(p));
    p.keys = keys;
    p.payload = payload;
    p.out_keys = out_keys;
    p.out_payload = out_payload;
    p.out_idx = out_idx;
    p.ws = static_cast<unsigned char*>(ws);
    p.n = n;
    p.base = base;
    const uint64_t vec = 16 / ks;
    uint64_t head = ((16 - (addr % 16)) % 16) / ks;
    if (head > n) head = n;
    if (qa.q) head = 0;  // topk_query: 16-byte aligned columns
    p.head = static_cast<uint32_t>(head);
    // query forms: the 4-byte columns' slabs need multiples of 4 rows (16 B) per copy
    p.body_n = qa.q ? n / 4 * 4 : (n - head) / vec * vec;
    const uint32_t tk = qa.q ? query_tile_keys(dtype, qa.q) : tile_keys_for(dtype);
    if (qa.q) {
        p.col_b = qa.rank_b;
        p.rank_w = qa.rank_w;
        if (qa.q & topk::kQPred) {
            p.pred = qa.pred.col;
            p.pred_in = qa.pred.kind == TOPK_PRED_IN ? 1u : 0u;
            p.pred_lo = qa.pred.lo;
            p.pred_span = qa.pred.hi > qa.pred.lo ? qa.pred.hi - qa.pred.lo : 0u;
            p.pred_mask = qa.pred.in_mask;
        }
    }
    const uint64_t ntiles = (p.body_n + tk - 1) / tk;
    p.ntiles = static_cast<uint32_t>(ntiles);
    p.k = k;
    p.K = next_pow2_u32(k);
    // Work blocks (tiles claimed together) and their permutation (2h bits cover them).
    p.blk = ntiles >= 16ull * static_cast<uint64_t>(sms) ? 8u : 1u;
    static const int blk_env = [] {
        const char* v = std::getenv("TOPK_BLOCK");
        return v ? std::atoi(v) : 0;
    }();
    if (blk_env > 0) p.blk = static_cast<uint32_t>(blk_env);
    p.nblocks = static_cast<uint32_t>((ntiles + p.blk - 1) / p.blk);
    static const int wave_env = [] {
        const char* v = std::getenv("TOPK_WAVE");
        return v ? std::atoi(v) : 0;
    }();
    // default: one block per SM per wave -- all SMs stream one address window at a
    // time (DRAM row locality), waves in pseudo-random order (robust to sorted input)
    p.wave = wave_env > 0 ? static_cast<uint32_t>(wave_env) : static_cast<uint32_t>(sms);
    p.nwaves = (p.nblocks + p.wave - 1) / p.wave;
    uint32_t bits = 0;
    while ((1ull << bits) < p.nwaves) ++bits;
    p.perm_h = p.nwaves > 1 ? (bits + 1) / 2 : 0;
    static const int perm_env = [] {
        const char* v = std::getenv("TOPK_PERM");
        return v ? std::atoi(v) : 1;
    }();
    if (!perm_env) p.perm_h = 0;
    const int grid = static_cast<int>(ntiles == 0 ? 1 : (ntiles < (uint64_t)sms ? ntiles : sms));
    p.gmax = static_cast<uint32_t>(sms);
    // Published samples: the 2^j-th best of each run for 2^j <= k (select.cuh flush).
    p.J = 0;
    while (p.J < static_cast<uint32_t>(topk::kPubRows) && (1u << p.J) <= k) ++p.J;

    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const bool mn = order == TOPK_SMALLEST, filt = mode == TOPK_MODE_FILTER;
    // Small inputs in filter mode run the pure kernel too: the result is identical, and
    // up to 2^22 keys (k <= 32) its fixed cost is lower than the streaming pass's (boot
    // flush, tail) -- graph-timed on B200, 2^20 keys k = 32: 36.9 -> 19.9 us (DESIGN.md
    // §4.4).  TOPK_PURE_SMALL_N overrides the cut (0 disables it).
    static const uint64_t small_cut = [] {
        const char* e = std::getenv("TOPK_PURE_SMALL_N");
        return e ? static_cast<uint64_t>(std::strtoull(e, nullptr, 10)) : (1ull << 22);
    }();
    const bool small_pure = filt && n <= small_cut;
    if (((!filt && p.K <= 256) || (small_pure && p.K <= 32)) && !qa.q && dtype != TOPK_F64) {
        // the paper's pure method, register/shuffle form (pure.cuh): 32-bit keys, K <= 256
        topk::PureParams pp;
        pp.keys = keys;
        pp.payload = payload;
        pp.out_keys = out_keys;
        pp.out_payload = out_payload;
        pp.out_idx = out_idx;
        pp.ticket = reinterpret_cast<unsigned int*>(p.ws) + 5;  // WsHeader::pad[0 .. 10]
        pp.cand = reinterpret_cast<uint64_t*>(p.ws + topk::ws_cand_offset(p.gmax));
        pp.n = n;
        pp.base = base;
        pp.k = k;
        pp.L = static_cast<uint32_t>(__builtin_ctz(p.K));
        // chunks are dealt round robin over the CTAs: up to one CTA per SM, one per chunk
        const uint64_t nch = (n + topk::kPureChunk - 1) / topk::kPureChunk;
        static const uint64_t grid_cap = [] {  // dev knob: TOPK_PURE_GRID (max CTAs)
            const char* e = std::getenv("TOPK_PURE_GRID");
            return e ? static_cast<uint64_t>(std::strtoull(e, nullptr, 10)) : 0ull;
        }();
        uint64_t cap = static_cast<uint64_t>(sms);
        // The merge tree above the CTAs costs a level per kPureGroup-fold of CTAs: up to
        // 16 chunks run in ONE CTA (no tree: 2^12 keys, k = 32, graph-timed 11.9 -> 8.6
        // us), up to 16 x 16 chunks in kPureGroup CTAs (one level); larger inputs spread
        // over every SM (fewer busy warps per SM: faster chunks)
        const uint64_t per_cta = static_cast<uint64_t>(topk::kPureNW);
        if (nch <= per_cta)
            cap = 1;
        else if (nch <= per_cta * topk::kPureGroup && cap > static_cast<uint64_t>(topk::kPureGroup))
            cap = topk::kPureGroup;
        if (grid_cap > 0 && grid_cap < cap) cap = grid_cap;
        const int pgrid = static_cast<int>(nch < cap ? nch : cap);
        const cudaError_t e = topk::launch_pure(key_kind(dtype), mn, pp, pgrid, st);
        if (e == cudaSuccess) g_launches.fetch_add(1, std::memory_order_relaxed);
        return e == cudaSuccess ? TOPK_OK : TOPK_ERR_CUDA;
    }
    if (qa.q & topk::kQKey2) {
        p.out_keys2 = qa.out_keys2;
        p.order2_min = qa.order2_min;
        p.col_c = qa.col_c;
        p.out_keys3 = qa.out_keys3;
        p.order3_min = qa.order3_min;
        return launch_variant((qa.q & topk::kQKey3) ? topk::kKeyKKK : topk::kKeyKK, mn, true, qa.q,
                              p, grid, st) == cudaSuccess
                   ? TOPK_OK : TOPK_ERR_CUDA;
    }
    return launch_variant(key_kind(dtype), mn, qa.q ? true : filt, qa.q, p, grid, st) == cudaSuccess
               ? TOPK_OK : TOPK_ERR_CUDA;
}


// Inputs longer than one launch indexes (32-bit local row ids): chunks of chunk_n() keys,
// each reduced by its own launch with its base offset (global ids), then the merge
// kernel -- the decomposition the paper uses across cores.

topk_status_t topk_select(topk_dtype_t dtype, const void* keys, const uint32_t* payload,
                          uint64_t n, uint64_t base, uint32_t k, topk_order_t order,
                          topk_mode_t mode, void* out_keys, uint32_t* out_payload,
                          int64_t* out_idx, void* ws, size_t ws_bytes, void* stream) {
    if (n <= kMaxLaunchN && n <= chunk_n())
        return select_one(dtype, keys, payload, n, base, k, order, mode, out_keys, out_payload,
                          out_idx, ws, ws_bytes, stream);
    // every argument error is reported before the first chunk is enqueued
    if (!valid_dtype(dtype) || !valid_order(order) || !keys || k == 0 || k > TOPK_MAX_K ||
        k > n)
        return TOPK_ERR_INVALID_ARG;
    if (mode != TOPK_MODE_FILTER && mode != TOPK_MODE_PURE) return TOPK_ERR_INVALID_ARG;
    if (out_payload && !payload) return TOPK_ERR_INVALID_ARG;
    if (reinterpret_cast<uintptr_t>(keys) % key_size(dtype)) return TOPK_ERR_INVALID_ARG;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return TOPK_ERR_CUDA;
    if (major != 10 || sms > topk::kGMax) return TOPK_ERR_UNSUPPORTED;
    const uint64_t nch = (n + chunk_n() - 1) / chunk_n();
    if (nch * k > 65536) return TOPK_ERR_UNSUPPORTED;
    const ChunkLayout L = chunk_layout(dtype, nch, k, sms);
    if (!ws || ws_bytes < L.total || (reinterpret_cast<uintptr_t>(ws) % 256))
        return TOPK_ERR_WORKSPACE;
    unsigned char* w = static_cast<unsigned char*>(ws);
    const size_t ks = key_size(dtype);
    uint64_t total = 0;
    for (uint64_t c = 0; c < nch; ++c) {
        const uint64_t lo = c * chunk_n(), len = (n - lo < chunk_n()) ? n - lo : chunk_n();
        const uint32_t kc = len < k ? static_cast<uint32_t>(len) : k;  // ragged last chunk
        topk_status_t st = select_one(
            dtype, static_cast<const unsigned char*>(keys) + lo * ks,
            payload ? payload + lo : nullptr, len, base + lo, kc, order, mode,
            w + L.ck + total * ks, payload ? reinterpret_cast<uint32_t*>(w + L.cp) + total : nullptr,
            reinterpret_cast<int64_t*>(w + L.ci) + total, w + L.sel, L.ck, stream);
        if (st != TOPK_OK) return st;
        total += kc;
    }
    // the chunks' results are sorted runs of k entries (the last one may be shorter)
    // chunks in order: chunk c's ids all below chunk c+1's
    return merge_total(dtype, w + L.ck, reinterpret_cast<const int64_t*>(w + L.ci),
                       payload ? reinterpret_cast<const uint32_t*>(w + L.cp) : nullptr, total, k,
                       true, k, order, out_keys, out_payload, out_idx, stream, true);
}

topk_status_t topk_query(topk_dtype_t dtype, const void* keys, const float* rank_b,
                         float rank_w, const topk_pred_t* pred, const uint32_t* payload,
                         uint64_t n, uint32_t k, topk_order_t order, void* out_keys,
                         uint32_t* out_payload, int64_t* out_idx, void* ws, size_t ws_bytes,
                         void* stream) {
    if (!valid_dtype(dtype) || !keys || n == 0 || n > kMaxLaunchN) return TOPK_ERR_INVALID_ARG;
    QueryArgs qa;
    if (rank_b) {
        if (dtype != TOPK_F32) return TOPK_ERR_INVALID_ARG;
        qa.q |= topk::kQRank;
        qa.rank_b = rank_b;
        qa.rank_w = rank_w;
    }
    if (pred) {
        if ((pred->kind != TOPK_PRED_RANGE && pred->kind != TOPK_PRED_IN) || !pred->col)
            return TOPK_ERR_INVALID_ARG;
        qa.q |= topk::kQPred;
        qa.pred = *pred;
    }
    if (!qa.q) return TOPK_ERR_INVALID_ARG;
    auto misaligned = [](const void* c) { return reinterpret_cast<uintptr_t>(c) % 16 != 0; };
    if (misaligned(keys) || (rank_b && misaligned(rank_b)) || (pred && misaligned(pred->col)) ||
        (payload && misaligned(payload)))
        return TOPK_ERR_INVALID_ARG;
    return select_one(dtype, keys, payload, n, 0, k, order, TOPK_MODE_FILTER, out_keys,
                      out_payload, out_idx, ws, ws_bytes, stream, qa);
}

topk_status_t topk_kk(const float* keys1, const float* keys2, const topk_pred_t* pred,
                      const uint32_t* payload, uint64_t n, uint32_t k, topk_order_t order1,
                      topk_order_t order2, float* out_keys1, float* out_keys2,
                      uint32_t* out_payload, int64_t* out_idx, void* ws, size_t ws_bytes,
                      void* stream) {
    if (!keys1 || !keys2 || n == 0 || n > kMaxLaunchN) return TOPK_ERR_INVALID_ARG;
    if (!valid_order(order1) || !valid_order(order2)) return TOPK_ERR_INVALID_ARG;
    QueryArgs qa;
    qa.q = topk::kQKey2;
    qa.rank_b = keys2;
    qa.out_keys2 = out_keys2;
    qa.order2_min = order2 == TOPK_SMALLEST ? 1u : 0u;
    if (pred) {
        if ((pred->kind != TOPK_PRED_RANGE && pred->kind != TOPK_PRED_IN) || !pred->col)
            return TOPK_ERR_INVALID_ARG;
        qa.q |= topk::kQPred;
        qa.pred = *pred;
    }
    auto misaligned = [](const void* c) { return reinterpret_cast<uintptr_t>(c) % 16 != 0; };
    if (misaligned(keys1) || misaligned(keys2) || (pred && misaligned(pred->col)) ||
        (payload && misaligned(payload)))
        return TOPK_ERR_INVALID_ARG;
    // 12-byte (64-bit code, row) entries: the f64 workspace layout
    return select_one(TOPK_F64, keys1, payload, n, 0, k, order1, TOPK_MODE_FILTER, out_keys1,
                      out_payload, out_idx, ws, ws_bytes, stream, qa);
}

// ---- radix-select top-k (radix.cuh; the paper's selection-based method) ----
struct RadixPlan {
    uint32_t G, cap;
    uint64_t slice;
};
static RadixPlan radix_plan(uint64_t n, int sms) {
    RadixPlan r;
    // 4 CTAs of 256 threads per SM, one contiguous slice each
    const uint64_t g = 4ull * static_cast<uint64_t>(sms);
    uint64_t slice = (n + g - 1) / g;
    slice = (slice + topk::kRadixTile - 1) / topk::kRadixTile * topk::kRadixTile;
    r.slice = slice;
    r.G = static_cast<uint32_t>((n + slice - 1) / slice);
    uint64_t cap = n / 16;
    if (cap < 65536) cap = 65536;
    if (cap > n) cap = n;
    r.cap = static_cast<uint32_t>(cap);
    return r;
}

size_t topk_radix_workspace_bytes(topk_dtype_t dtype, uint64_t n, uint32_t k) {
    if (!valid_dtype(dtype) || n == 0 || k == 0 || k > TOPK_MAX_K || k > n || n > kMaxLaunchN)
        return 0;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return 0;
    const RadixPlan r = radix_plan(n, sms);
    return topk::radix_workspace_bytes(key_kind(dtype), r.G, k, r.cap);
}

topk_status_t topk_radix(topk_dtype_t dtype, const void* keys, uint64_t n, uint32_t k,
                         topk_order_t order, void* out_keys, int64_t* out_idx, void* ws,
                         size_t ws_bytes, void* stream) {
    if (!valid_dtype(dtype) || !valid_order(order)) return TOPK_ERR_INVALID_ARG;
    if (!keys || n == 0 || k == 0 || k > TOPK_MAX_K || k > n || n > kMaxLaunchN)
        return TOPK_ERR_INVALID_ARG;
    if (reinterpret_cast<uintptr_t>(keys) % key_size(dtype)) return TOPK_ERR_INVALID_ARG;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return TOPK_ERR_CUDA;
    if (major != 10) return TOPK_ERR_UNSUPPORTED;
    const RadixPlan r = radix_plan(n, sms);
    if (!ws || (reinterpret_cast<uintptr_t>(ws) % 256) ||
        ws_bytes < topk::radix_workspace_bytes(key_kind(dtype), r.G, k, r.cap))
        return TOPK_ERR_WORKSPACE;
    topk::RadixParams p;
    std::memset(&p, 0, sizeof(p));
    p.keys = keys;
    p.n = n;
    p.base = 0;
    p.k = k;
    p.K = next_pow2_u32(k);
    p.G = r.G;
    p.slice = r.slice;
    p.cap = r.cap;
    p.ws = static_cast<unsigned char*>(ws);
    p.out_keys = out_keys;
    p.out_idx = out_idx;
    int launches = 0;
    const cudaError_t e = topk::launch_radix(key_kind(dtype), order == TOPK_SMALLEST, p,
                                             static_cast<cudaStream_t>(stream), &launches);
    if (e != cudaSuccess) return TOPK_ERR_CUDA;
    g_launches.fetch_add(static_cast<uint64_t>(launches), std::memory_order_relaxed);
    return TOPK_OK;
}

topk_status_t topk_kkk(const float* keys1, const float* keys2, const float* keys3,
                       const topk_pred_t* pred, const uint32_t* payload, uint64_t n, uint32_t k,
                       topk_order_t order1, topk_order_t order2, topk_order_t order3,
                       float* out_keys1, float* out_keys2, float* out_keys3,
                       uint32_t* out_payload, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream) {
    if (!keys1 || !keys2 || !keys3 || n == 0 || n > kMaxLaunchN) return TOPK_ERR_INVALID_ARG;
    if (!valid_order(order1) || !valid_order(order2) || !valid_order(order3))
        return TOPK_ERR_INVALID_ARG;
    QueryArgs qa;
    qa.q = topk::kQKey2 | topk::kQKey3;
    qa.rank_b = keys2;
    qa.out_keys2 = out_keys2;
    qa.order2_min = order2 == TOPK_SMALLEST ? 1u : 0u;
    qa.col_c = keys3;
    qa.out_keys3 = out_keys3;
    qa.order3_min = order3 == TOPK_SMALLEST ? 1u : 0u;
    if (pred) {
        if ((pred->kind != TOPK_PRED_RANGE && pred->kind != TOPK_PRED_IN) || !pred->col)
            return TOPK_ERR_INVALID_ARG;
        qa.q |= topk::kQPred;
        qa.pred = *pred;
    }
    auto misaligned = [](const void* c) { return reinterpret_cast<uintptr_t>(c) % 16 != 0; };
    if (misaligned(keys1) || misaligned(keys2) || misaligned(keys3) ||
        (pred && misaligned(pred->col)) || (payload && misaligned(payload)))
        return TOPK_ERR_INVALID_ARG;
    return select_one(TOPK_F64, keys1, payload, n, 0, k, order1, TOPK_MODE_FILTER, out_keys1,
                      out_payload, out_idx, ws, ws_bytes, stream, qa);
}

topk_status_t topk_f32(const float* keys, uint64_t n, uint32_t k, topk_order_t order,
                       float* out_keys, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream) {
    return topk_select(TOPK_F32, keys, nullptr, n, 0, k, order, TOPK_MODE_FILTER, out_keys,
                       nullptr, out_idx, ws, ws_bytes, stream);
}
topk_status_t topk_u32(const uint32_t* keys, uint64_t n, uint32_t k, topk_order_t order,
                       uint32_t* out_keys, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream) {
    return topk_select(TOPK_U32, keys, nullptr, n, 0, k, order, TOPK_MODE_FILTER, out_keys,
                       nullptr, out_idx, ws, ws_bytes, stream);
}
topk_status_t topk_f64(const double* keys, uint64_t n, uint32_t k, topk_order_t order,
                       double* out_keys, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream) {
    return topk_select(TOPK_F64, keys, nullptr, n, 0, k, order, TOPK_MODE_FILTER, out_keys,
                       nullptr, out_idx, ws, ws_bytes, stream);
}
topk_status_t topk_u32_kv(const uint32_t* keys, const uint32_t* payload, uint64_t n,
                          uint32_t k, topk_order_t order, uint32_t* out_keys,
                          uint32_t* out_payload, int64_t* out_idx, void* ws,
                          size_t ws_bytes, void* stream) {
    return topk_select(TOPK_U32, keys, payload, n, 0, k, order, TOPK_MODE_FILTER, out_keys,
                       out_payload, out_idx, ws, ws_bytes, stream);
}
topk_status_t topk_f64_kv(const double* keys, const uint32_t* payload, uint64_t n,
                          uint32_t k, topk_order_t order, double* out_keys,
                          uint32_t* out_payload, int64_t* out_idx, void* ws,
                          size_t ws_bytes, void* stream) {
    return topk_select(TOPK_F64, keys, payload, n, 0, k, order, TOPK_MODE_FILTER, out_keys,
                       out_payload, out_idx, ws, ws_bytes, stream);
}

size_t topk_merge_workspace_bytes(topk_dtype_t dtype, uint32_t runs, uint32_t run_len,
                                  uint32_t k) {
    (void)dtype;
    (void)runs;
    (void)run_len;
    (void)k;
    return 256;  // the merge runs in one CTA's shared memory; reserved for future use
}

topk_status_t topk_merge(topk_dtype_t dtype, const void* cand_keys, const int64_t* cand_idx,
                         const uint32_t* cand_payload, uint32_t runs, uint32_t run_len,
                         uint32_t k, topk_order_t order, void* out_keys,
                         uint32_t* out_payload, int64_t* out_idx, void* ws,
                         size_t ws_bytes, void* stream) {
    (void)ws;
    (void)ws_bytes;
    if (runs == 0 || run_len == 0) return TOPK_ERR_INVALID_ARG;
    return merge_total(dtype, cand_keys, cand_idx, cand_payload,
                       static_cast<uint64_t>(runs) * run_len, run_len, false, k, order, out_keys,
                       out_payload, out_idx, stream);
}

topk_status_t topk_merge_sorted(topk_dtype_t dtype, const void* cand_keys,
                                const int64_t* cand_idx, const uint32_t* cand_payload,
                                uint32_t runs, uint32_t run_len, uint32_t k, topk_order_t order,
                                void* out_keys, uint32_t* out_payload, int64_t* out_idx,
                                void* ws, size_t ws_bytes, void* stream) {
    (void)ws;
    (void)ws_bytes;
    if (runs == 0 || run_len == 0) return TOPK_ERR_INVALID_ARG;
    return merge_total(dtype, cand_keys, cand_idx, cand_payload,
                       static_cast<uint64_t>(runs) * run_len, run_len, true, k, order, out_keys,
                       out_payload, out_idx, stream);
}

/* Debug (not in topk.h's stable surface): read / reset the device counters of
 * select_kernel (flushes, survivors flushed, flush cycles, deferrals, tiles). */
int topk_debug_stats(uint64_t* host8, int reset) {
    // (a variant build may compile only some select TUs with -DTOPK_DEBUG: the others
    // have no counters and are skipped)
    for (int i = 0; i < 8; ++i) host8[i] = 0;
    int found = 0;
    for (int i = 0; i < topk::kSelectTableN; ++i) {
        const auto f = topk::kSelectTable[i].debug;
        if (f(topk::kDbgStatsAdd, host8, 0) != 0) continue;
        if (reset && f(topk::kDbgStatsReset, nullptr, 0) != 0) return -1;
        ++found;
    }
    return found ? 0 : -1;
}

topk_status_t topk_probe_read(const void* data, size_t bytes, int method, int grid, int tile,
                              int stages, uint32_t* sink, void* stream) {
    if (!data || !sink || bytes == 0 || (bytes % 16) || (reinterpret_cast<uintptr_t>(data) % 16))
        return TOPK_ERR_INVALID_ARG;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return TOPK_ERR_CUDA;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (method == 0) {
        const int g = grid > 0 ? grid : 4 * sms;
        topk::probe_ldg_kernel<<<g, 512, 0, st>>>(static_cast<const uint4*>(data), bytes / 16,
                                                  sink);
    } else if (method == 1) {
        if (tile <= 0 || (tile % 16) || stages <= 0) return TOPK_ERR_INVALID_ARG;
        const size_t smem = static_cast<size_t>(tile) * stages + 16 * static_cast<size_t>(stages);
        if (smem > 227 * 1024) return TOPK_ERR_INVALID_ARG;
        if (cudaFuncSetAttribute(topk::probe_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 static_cast<int>(smem)) != cudaSuccess)
            return TOPK_ERR_CUDA;
        const int g = grid > 0 ? grid : sms;
        topk::probe_tma_kernel<<<g, 512, smem, st>>>(static_cast<const unsigned char*>(data),
                                                     bytes, tile, stages, sink);
    } else {
        return TOPK_ERR_INVALID_ARG;
    }
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return cudaGetLastError() == cudaSuccess ? TOPK_OK : TOPK_ERR_CUDA;
}

/* Debug: the code-only network (cnet.cuh) on n <= 4096 device codes (u32, or u64 if
 * e64), 4 <= Lp <= 9; d_out receives the top-2^Lp codes best first. */
int topk_debug_cnet(int e64, const void* d_codes, int n, int Lp, void* d_out) {
    if (n < 1 || n > 4096 || Lp < 4 || Lp > 9) return -1;
    const size_t smem = 4096 * 12 + 4096 * 8;
    if (e64) {
        cudaFuncSetAttribute(topk::cnet_debug_kernel<topk::E64, 15>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        topk::cnet_debug_kernel<topk::E64, 15><<<1, 480, smem>>>(
            static_cast<const uint64_t*>(d_codes), n, Lp, static_cast<uint64_t*>(d_out));
    } else {
        cudaFuncSetAttribute(topk::cnet_debug_kernel<topk::E32, 15>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        topk::cnet_debug_kernel<topk::E32, 15><<<1, 480, smem>>>(
            static_cast<const uint32_t*>(d_codes), n, Lp, static_cast<uint32_t*>(d_out));
    }
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return cudaDeviceSynchronize() == cudaSuccess ? 0 : -1;
}

/* Debug switches of the select kernel (select.cuh c_dbg), set in every select TU. */
int topk_debug_flags(int flags) {
    for (int i = 0; i < topk::kSelectTableN; ++i)
        if (topk::kSelectTable[i].debug(topk::kDbgFlags, nullptr, flags) != 0) return -1;
    return 0;
}

/* Debug timeline (see select.cuh g_trace): enable=1 clears and enables, 0 disables;
 * copies kTraceCtas x kTraceLen u64 to host (may be NULL) -- per CTA row, from the
 * select TU that recorded events (one key type is traced at a time). */
int topk_debug_trace(int enable, uint64_t* host) {
    constexpr size_t kRows = topk::kTraceCtas, kLen = topk::kTraceLen;
    if (host) {
        static uint64_t tmp[kRows * kLen];
        std::memset(host, 0, sizeof(tmp));
        for (int i = 0; i < topk::kSelectTableN; ++i) {
            if (topk::kSelectTable[i].debug(topk::kDbgTraceRead, tmp, 0) != 0) return -1;
            for (size_t r = 0; r < kRows; ++r)
                if (tmp[r * kLen] > host[r * kLen])
                    std::memcpy(host + r * kLen, tmp + r * kLen, kLen * sizeof(uint64_t));
        }
    }
    for (int i = 0; i < topk::kSelectTableN; ++i)
        if (topk::kSelectTable[i].debug(topk::kDbgTraceSet, nullptr, enable) != 0) return -1;
    return 0;
}

// ---- host-resident input: chunked H2D overlapped with the reductive pass ----
struct HostLayout {
    size_t stage[2], ck, ci, sel, ok, oi, total;
};
static HostLayout host_layout(topk_dtype_t dtype, uint64_t n, uint32_t k, uint64_t chunk,
                              int sms) {
    const size_t ks = key_size(dtype);
    const uint64_t nch = (n + chunk - 1) / chunk;
    HostLayout L;
    L.stage[0] = 0;
    L.stage[1] = align_up(chunk * ks, 256);
    L.ck = L.stage[1] + align_up(chunk * ks, 256);
    L.ci = L.ck + align_up(nch * k * ks, 256);
    L.sel = L.ci + align_up(nch * k * 8, 256);
    L.ok = L.sel + align_up(select_ws_bytes(dtype, k, sms), 256);
    L.oi = L.ok + align_up(k * ks, 256);
    L.total = L.oi + align_up(k * 8, 256);
    return L;
}

size_t topk_host_workspace_bytes(topk_dtype_t dtype, uint64_t n, uint32_t k,
                                 uint64_t chunk_keys) {
    if (!valid_dtype(dtype) || n == 0 || k == 0 || k > TOPK_MAX_K || k > n) return 0;
    if (chunk_keys < 4096 || (chunk_keys % 4) || chunk_keys > kMaxLaunchN) return 0;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return 0;
    return host_layout(dtype, n, k, chunk_keys, sms).total;
}

topk_status_t topk_select_host(topk_dtype_t dtype, const void* h_keys, uint64_t n, uint32_t k,
                               topk_order_t order, void* h_out_keys, int64_t* h_out_idx,
                               uint64_t chunk_keys, void* ws, size_t ws_bytes, void* stream) {
    if (!valid_dtype(dtype) || !valid_order(order) || !h_keys) return TOPK_ERR_INVALID_ARG;
    if (n == 0 || k == 0 || k > TOPK_MAX_K || k > n) return TOPK_ERR_INVALID_ARG;
    if (chunk_keys < 4096 || (chunk_keys % 4) || chunk_keys > kMaxLaunchN)
        return TOPK_ERR_INVALID_ARG;
    const uint64_t nch = (n + chunk_keys - 1) / chunk_keys;
    if (nch * k > 65536) return TOPK_ERR_INVALID_ARG;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return TOPK_ERR_CUDA;
    const HostLayout L = host_layout(dtype, n, k, chunk_keys, sms);
    if (!ws || ws_bytes < L.total || (reinterpret_cast<uintptr_t>(ws) % 256))
        return TOPK_ERR_WORKSPACE;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev >= 64) return TOPK_ERR_CUDA;
    // library-owned copy stream + events, one set per device
    static cudaStream_t copy_st[64];
    static cudaEvent_t copied[64][2], freed[64][2], start[64];
    if (!copy_st[dev]) {
        if (cudaStreamCreateWithFlags(&copy_st[dev], cudaStreamNonBlocking) != cudaSuccess)
            return TOPK_ERR_CUDA;
        for (int b = 0; b < 2; ++b) {
            cudaEventCreateWithFlags(&copied[dev][b], cudaEventDisableTiming);
            cudaEventCreateWithFlags(&freed[dev][b], cudaEventDisableTiming);
        }
        cudaEventCreateWithFlags(&start[dev], cudaEventDisableTiming);
    }
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaStream_t cp = copy_st[dev];
    unsigned char* w = static_cast<unsigned char*>(ws);
    const size_t ks = key_size(dtype);
    // the staging buffers may still be read by earlier work on `stream`
    if (cudaEventRecord(start[dev], st) != cudaSuccess) return TOPK_ERR_CUDA;
    cudaStreamWaitEvent(cp, start[dev], 0);
    uint64_t total = 0;
    for (uint64_t c = 0; c < nch; ++c) {
        const int b = static_cast<int>(c & 1);
        const uint64_t lo = c * chunk_keys;
        const uint64_t len = (n - lo < chunk_keys) ? n - lo : chunk_keys;
        if (c >= 2) cudaStreamWaitEvent(cp, freed[dev][b], 0);
        if (cudaMemcpyAsync(w + L.stage[b], static_cast<const unsigned char*>(h_keys) + lo * ks,
                            len * ks, cudaMemcpyHostToDevice, cp) != cudaSuccess)
            return TOPK_ERR_CUDA;
        cudaEventRecord(copied[dev][b], cp);
        cudaStreamWaitEvent(st, copied[dev][b], 0);
        const uint32_t kc = len < k ? static_cast<uint32_t>(len) : k;  // ragged last chunk
        topk_status_t r = select_one(dtype, w + L.stage[b], nullptr, len, lo, kc, order,
                                     TOPK_MODE_FILTER, w + L.ck + total * ks, nullptr,
                                     reinterpret_cast<int64_t*>(w + L.ci) + total, w + L.sel,
                                     L.ok - L.sel, stream);
        if (r != TOPK_OK) return r;
        cudaEventRecord(freed[dev][b], st);
        total += kc;
    }
    topk_status_t r = merge_total(dtype, w + L.ck, reinterpret_cast<const int64_t*>(w + L.ci),
                                  nullptr, total, k, true, k, order, w + L.ok, nullptr,
                                  reinterpret_cast<int64_t*>(w + L.oi), stream, true);
    if (r != TOPK_OK) return r;
    if (h_out_keys &&
        cudaMemcpyAsync(h_out_keys, w + L.ok, k * ks, cudaMemcpyDeviceToHost, st) != cudaSuccess)
        return TOPK_ERR_CUDA;
    if (h_out_idx &&
        cudaMemcpyAsync(h_out_idx, w + L.oi, k * 8, cudaMemcpyDeviceToHost, st) != cudaSuccess)
        return TOPK_ERR_CUDA;
    return cudaGetLastError() == cudaSuccess ? TOPK_OK : TOPK_ERR_CUDA;
}

uint64_t topk_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

const char* topk_status_string(topk_status_t s) {
    switch (s) {
        case TOPK_OK: return "TOPK_OK";
        case TOPK_ERR_INVALID_ARG: return "TOPK_ERR_INVALID_ARG: invalid argument";
        case TOPK_ERR_UNSUPPORTED: return "TOPK_ERR_UNSUPPORTED: device or size not supported";
        case TOPK_ERR_WORKSPACE: return "TOPK_ERR_WORKSPACE: workspace NULL, too small or misaligned";
        case TOPK_ERR_CUDA: return "TOPK_ERR_CUDA: CUDA runtime or launch error";
        case TOPK_ERR_NCCL: return "TOPK_ERR_NCCL: NCCL call failed";
    }
    return "unknown topk_status_t";
}

int topk_abi_version(void) { return TOPK_ABI_VERSION; }

}  // extern "C"

static topk_status_t merge_total(topk_dtype_t dtype, const void* cand_keys,
                                 const int64_t* cand_idx, const uint32_t* cand_payload,
                                 uint64_t total, uint32_t run_len, bool sorted, uint32_t k,
                                 topk_order_t order, void* out_keys, uint32_t* out_payload,
                                 int64_t* out_idx, void* stream, bool ordered,
                                 const uint64_t* ranges) {
    if (!valid_dtype(dtype) || !valid_order(order)) return TOPK_ERR_INVALID_ARG;
    if (!cand_keys || !cand_idx || total == 0) return TOPK_ERR_INVALID_ARG;
    if (total > 65536 || k == 0 || k > TOPK_MAX_K || k > total) return TOPK_ERR_INVALID_ARG;
    if (out_payload && !cand_payload) return TOPK_ERR_INVALID_ARG;
    int sms = 0, major = 0;
    if (!device_info(&sms, &major)) return TOPK_ERR_CUDA;
    if (major != 10) return TOPK_ERR_UNSUPPORTED;
    topk::MergeParams p;
    p.cand_keys = cand_keys;
    p.cand_idx = cand_idx;
    p.cand_payload = cand_payload;
    p.out_keys = out_keys;
    p.out_payload = out_payload;
    p.out_idx = out_idx;
    p.total = static_cast<uint32_t>(total);
    p.run_len = run_len == 0 ? 1u : run_len;
    p.sorted = sorted ? 1u : 0u;
    p.ordered = sorted ? (ordered ? 1u : (ranges ? 0u : 2u)) : 0u;
    p.ranges = sorted ? ranges : nullptr;
    p.k = k;
    p.K = next_pow2_u32(k);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const bool mn = order == TOPK_SMALLEST;
    cudaError_t e;
    switch (dtype) {
        case TOPK_F32: e = dispatch_merge<float>(p, mn, st); break;
        case TOPK_U32: e = dispatch_merge<uint32_t>(p, mn, st); break;
        default: e = dispatch_merge<double>(p, mn, st); break;
    }
    return e == cudaSuccess ? TOPK_OK : TOPK_ERR_CUDA;
}

#include "sharded.cuh"
