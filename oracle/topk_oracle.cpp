/*
 * oracle/topk_oracle.cpp -- CPU ORACLE for bitonic top-k.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product path (paper_conf_sigmod_shanbhagpm18_b200)
 * never links, imports or calls it; it shares no header, table or helper with the CUDA
 * path.
 *
 * What it computes -- the plain definition, not a simulation of the algorithm:
 * the paper's bitonic top-k is exact ("we know that the top-k elements were selected",
 * PAPER.md P:150 §3.2(2); "performs no unnecessary work"), so its result is the
 * first k elements of the input under a total order.  The problem statement is
 * "find the top-k items, i.e., the largest or smallest ... (ORDER BY / LIMIT)"
 * (P:16 Abstract) and "the highest (or lowest) k of n tuples" (§1).
 *
 * Total order (readings R1-R4; the paper is silent on ties, NaN and +-0):
 *   better(a, b) := code(a) > code(b) || (code(a) == code(b) && idx(a) < idx(b))
 *   code(): f32/f64 -> order-preserving unsigned image; every NaN maps to the greatest
 *   code (NaN ranks above +inf and all NaNs are equal); -0 and +0 share one code;
 *   u32 -> the value itself.  Min order (ORDER BY ... ASC) complements the code, so
 *   the tie rule (lowest source index first) is the same in both orders.
 *   Output: best first, out_keys[j] is the original bit pattern of keys[out_idx[j]].
 *
 * Algorithm (the per-partition scheme the paper describes for CPU cores, §1 and
 * P:444 App. C): split the n (code, idx) pairs into P contiguous chunks; each thread
 * std::partial_sort's its chunk to its best k; one final std::partial_sort over the
 * P*k winners.  Exact because top-k decomposes under a strict total order.
 *
 * Also: oracle_certificate(), an O(n) check independent of partial_sort,
 * and oracle_query(), the database form of §5: WHERE predicate, ORDER BY a
 * ranking function, LIMIT k -- computed the unfused way the paper starts from ("a
 * separate kernel execute[s] the filter and ... the subsequent top-k kernel use[s] the
 * output"; "a separate projection step which outputs the value of the
 * function"): filter rows, project f, then the top-k above.
 */
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>
#include <sched.h>

namespace {

enum { DT_F32 = 0, DT_U32 = 1, DT_F64 = 2 };
enum { ORDER_LARGEST = 0, ORDER_SMALLEST = 1 };

struct Pair {
    uint64_t code;  // order code, larger = better (already complemented for min order)
    uint64_t idx;   // source index (the tie-break)
    uint64_t row;   // position inside the keys array (for the output gather)
};

// better(a, b): DESIGN.md reading R1 (ties -> lowest source index).
inline bool better(const Pair& a, const Pair& b) {
    if (a.code != b.code) return a.code > b.code;
    return a.idx < b.idx;
}

// Order code of one key (reading R2: NaN greatest, -0 == +0).
// Written from the IEEE-754 layout: for non-negative floats the bit pattern grows with
// the value; for negative floats it shrinks, so it is complemented; the sign-bit flip of
// non-negative patterns puts all of them above all negative ones.
uint64_t code_of(int dtype, const void* keys, uint64_t i, int order) {
    uint64_t c = 0;
    if (dtype == DT_F32) {
        float x;
        std::memcpy(&x, static_cast<const char*>(keys) + 4 * i, 4);
        uint32_t u;
        std::memcpy(&u, &x, 4);
        if (std::isnan(x)) {
            c = 0xFFFFFFFFu;
        } else if (x == 0.0f) {
            c = 0x80000000u;  // both zeros
        } else if (u >> 31) {
            c = (uint32_t)~u;
        } else {
            c = u | 0x80000000u;
        }
        if (order == ORDER_SMALLEST) c = (uint32_t)~(uint32_t)c;
    } else if (dtype == DT_F64) {
        double x;
        std::memcpy(&x, static_cast<const char*>(keys) + 8 * i, 8);
        uint64_t u;
        std::memcpy(&u, &x, 8);
        if (std::isnan(x)) {
            c = ~0ull;
        } else if (x == 0.0) {
            c = 0x8000000000000000ull;
        } else if (u >> 63) {
            c = ~u;
        } else {
            c = u | 0x8000000000000000ull;
        }
        if (order == ORDER_SMALLEST) c = ~c;
    } else {
        uint32_t u;
        std::memcpy(&u, static_cast<const char*>(keys) + 4 * i, 4);
        c = u;
        if (order == ORDER_SMALLEST) c = (uint32_t)~u;
    }
    return c;
}

int host_threads(int requested) {
    if (requested > 0) return requested;
    cpu_set_t set;
    CPU_ZERO(&set);
    if (sched_getaffinity(0, sizeof(set), &set) == 0) {
        int c = CPU_COUNT(&set);
        if (c > 0) return c;
    }
    unsigned h = std::thread::hardware_concurrency();
    return h ? (int)h : 1;
}

size_t key_bytes(int dtype) { return dtype == DT_F64 ? 8 : 4; }

// Per-partition top-k of rows [lo, hi): P:34 / P:444 "each processor computes a
// per-partition top-k".  idx_in (optional) supplies explicit source indices.
void chunk_topk(int dtype, const void* keys, const int64_t* idx_in, uint64_t base,
                uint64_t lo, uint64_t hi, uint32_t k, int order, std::vector<Pair>* out) {
    std::vector<Pair> v;
    v.reserve(hi - lo);
    for (uint64_t i = lo; i < hi; ++i) {
        Pair p;
        p.code = code_of(dtype, keys, i, order);
        p.idx = idx_in ? (uint64_t)idx_in[i] : base + i;
        p.row = i;
        v.push_back(p);
    }
    size_t kk = std::min<size_t>(k, v.size());
    std::partial_sort(v.begin(), v.begin() + kk, v.end(), better);
    v.resize(kk);
    out->swap(v);
}

}  // namespace

extern "C" {

/* Top-k of n keys (optional explicit indices idx_in[n]; else idx = base + i).
 * Writes out_keys[k] (original key bits, may be NULL) and out_idx[k] (may be NULL).
 * Returns the number of threads used, or -1 on an argument error. */
int oracle_topk(int dtype, const void* keys, const int64_t* idx_in, uint64_t n,
                uint64_t base, uint32_t k, int order, void* out_keys, int64_t* out_idx,
                int threads) {
    if (!keys || n == 0 || k == 0 || k > n) return -1;
    if (dtype < 0 || dtype > 2 || (order != 0 && order != 1)) return -1;
    int P = host_threads(threads);
    if ((uint64_t)P > n / 4096 + 1) P = (int)(n / 4096 + 1);  // tiny inputs: 1 chunk
    std::vector<std::vector<Pair>> part(P);
    std::vector<std::thread> th;
    uint64_t per = (n + P - 1) / P;
    for (int t = 0; t < P; ++t) {
        uint64_t lo = std::min<uint64_t>(n, per * t), hi = std::min<uint64_t>(n, lo + per);
        th.emplace_back(chunk_topk, dtype, keys, idx_in, base, lo, hi, k, order, &part[t]);
    }
    for (auto& x : th) x.join();
    // Global step: partial_sort over the P*k winners.
    std::vector<Pair> all;
    for (auto& p : part) all.insert(all.end(), p.begin(), p.end());
    std::partial_sort(all.begin(), all.begin() + k, all.end(), better);
    size_t kb = key_bytes(dtype);
    for (uint32_t j = 0; j < k; ++j) {
        uint64_t row = all[j].row;
        if (out_idx) out_idx[j] = (int64_t)all[j].idx;
        if (out_keys) std::memcpy(static_cast<char*>(out_keys) + kb * j,
                                  static_cast<const char*>(keys) + kb * row, kb);
    }
    return P;
}

/* O(n) certificate (SURVEY §8(c) "What pins each part"), independent of partial_sort:
 * given a claimed result (out_keys[k], out_idx[k], idx = base + row), returns 0 iff
 *  (i)  out is strictly decreasing under better(),
 *  (ii) every out_idx is in range and out_keys[j] is bit-identical to keys[out_idx[j]-base],
 *  (iii) exactly k-1 inputs are better than out[k-1],
 * which together imply out == the top-k.  Returns 1, 2 or 3 for the failed condition. */
int oracle_certificate(int dtype, const void* keys, uint64_t n, uint64_t base, uint32_t k,
                       int order, const void* out_keys, const int64_t* out_idx) {
    if (!keys || !out_keys || !out_idx || k == 0 || k > n) return -1;
    size_t kb = key_bytes(dtype);
    std::vector<Pair> o(k);
    for (uint32_t j = 0; j < k; ++j) {
        int64_t r = out_idx[j] - (int64_t)base;
        if (out_idx[j] < (int64_t)base || (uint64_t)r >= n) return 2;
        if (std::memcmp(static_cast<const char*>(out_keys) + kb * j,
                        static_cast<const char*>(keys) + kb * (uint64_t)r, kb) != 0)
            return 2;
        o[j].code = code_of(dtype, keys, (uint64_t)r, order);
        o[j].idx = (uint64_t)out_idx[j];
    }
    for (uint32_t j = 1; j < k; ++j)
        if (!better(o[j - 1], o[j])) return 1;  // strict => indices also distinct
    uint64_t cnt = 0;
    const Pair last = o[k - 1];
    for (uint64_t i = 0; i < n; ++i) {
        Pair p;
        p.code = code_of(dtype, keys, i, order);
        p.idx = base + i;
        p.row = i;
        if (better(p, last)) ++cnt;
    }
    return cnt == (uint64_t)(k - 1) ? 0 : 3;
}

/* Query form (queries 1-3 of §6.8):
 *   SELECT row, f(row) WHERE pred(row) ORDER BY f DESC|ASC LIMIT k
 * pred (reading R17): kind 0 none; 1 range lo <= pcol[i] < hi; 2 membership
 *   pcol[i] < 64 and bit pcol[i] of in_mask set (an IN list over a dictionary-coded
 *   column, e.g. "lang = 'en' OR lang = 'es'").
 * f (reading R18): rank_b == NULL -> f = keys[i] (any dtype); else (f32 only)
 *   f = keys[i] + w * rank_b[i], the product and the sum each rounded to float
 *   ("retweet_count + 0.5 * likes_count"; built with -ffp-contract=off); a NaN
 *   result is returned as the canonical quiet NaN 0x7FC00000 (IEEE-754 leaves the
 *   payload of a computed NaN open; it ranks the same either way).
 * Plain plan: (1) filter + project into a new array with the source row ids, (2)
 * oracle_topk over it with explicit indices.  Rows beyond the number of matches get
 * out_idx = -1 and all-zero key bits.  Returns the number of result rows (<= k), or
 * -1 on an argument error. */
int oracle_query(int dtype, const void* keys, const float* rank_b, float w, int pred_kind,
                 const uint32_t* pcol, uint32_t lo, uint32_t hi, uint64_t in_mask, uint64_t n,
                 uint32_t k, int order, void* out_keys, int64_t* out_idx, int threads) {
    if (!keys || n == 0 || k == 0 || dtype < 0 || dtype > 2) return -1;
    if (rank_b && dtype != DT_F32) return -1;
    if (pred_kind < 0 || pred_kind > 2 || (pred_kind && !pcol)) return -1;
    const size_t kb = key_bytes(dtype);
    std::vector<unsigned char> fk;
    std::vector<int64_t> fi;
    fk.reserve(n * kb);
    fi.reserve(n);
    for (uint64_t i = 0; i < n; ++i) {
        if (pred_kind == 1 && !(lo <= pcol[i] && pcol[i] < hi)) continue;
        if (pred_kind == 2 && !(pcol[i] < 64 && ((in_mask >> pcol[i]) & 1ull))) continue;
        unsigned char b[8];
        if (rank_b) {
            float a;
            std::memcpy(&a, static_cast<const char*>(keys) + 4 * i, 4);
            const float prod = w * rank_b[i];
            const float f = a + prod;
            std::memcpy(b, &f, 4);
            if (std::isnan(f)) {  // R18: a computed NaN is returned as the canonical 0x7FC00000
                const uint32_t qnan = 0x7FC00000u;
                std::memcpy(b, &qnan, 4);
            }
        } else {
            std::memcpy(b, static_cast<const char*>(keys) + kb * i, kb);
        }
        fk.insert(fk.end(), b, b + kb);
        fi.push_back(static_cast<int64_t>(i));
    }
    const uint64_t m = fi.size();
    const uint32_t kk = m < k ? static_cast<uint32_t>(m) : k;
    if (out_keys) std::memset(out_keys, 0, kb * k);
    if (out_idx)
        for (uint32_t j = 0; j < k; ++j) out_idx[j] = -1;
    if (kk > 0 && oracle_topk(dtype, fk.data(), fi.data(), m, 0, kk, order, out_keys, out_idx,
                              threads) < 0)
        return -1;
    return static_cast<int>(kk);
}

/* Compound keys (§6.6 "two keys + value (KKV)"; reading R19):
 *   ORDER BY k1 [DESC|ASC], k2 [DESC|ASC] LIMIT k  over two f32 columns
 * -- lexicographic: k1 decides, k2 breaks k1 ties, then the lowest row id.  Each
 * column's order is that of oracle_topk's code map (order1 / order2).  The compare is
 * written as the plain lexicographic rule on the two codes (no packing), and the
 * value (payload) is the tuple id gathered at the end.  Writes out_k1[k],
 * out_k2[k] (original bits), out_idx[k]; returns 0 or -1 on an argument error. */
int oracle_topk_kk(const float* k1, const float* k2, uint64_t n, uint32_t k, int order1,
                   int order2, float* out_k1, float* out_k2, int64_t* out_idx) {
    if (!k1 || !k2 || n == 0 || k == 0 || k > n) return -1;
    if ((order1 != 0 && order1 != 1) || (order2 != 0 && order2 != 1)) return -1;
    struct Row {
        uint64_t c1, c2, idx;
    };
    std::vector<Row> v(n);
    for (uint64_t i = 0; i < n; ++i) {
        v[i].c1 = code_of(DT_F32, k1, i, order1);
        v[i].c2 = code_of(DT_F32, k2, i, order2);
        v[i].idx = i;
    }
    auto lex_better = [](const Row& a, const Row& b) {
        if (a.c1 != b.c1) return a.c1 > b.c1;
        if (a.c2 != b.c2) return a.c2 > b.c2;
        return a.idx < b.idx;
    };
    std::partial_sort(v.begin(), v.begin() + k, v.end(), lex_better);
    for (uint32_t j = 0; j < k; ++j) {
        const uint64_t r = v[j].idx;
        if (out_idx) out_idx[j] = static_cast<int64_t>(r);
        if (out_k1) std::memcpy(out_k1 + j, k1 + r, 4);
        if (out_k2) std::memcpy(out_k2 + j, k2 + r, 4);
    }
    return 0;
}

/* Three compound keys -- "three keys + value (KKKV)" (§6.6; R19):
 * ORDER BY k1, k2, k3 LIMIT k, lexicographic on the three columns' codes, then the
 * lowest row id (the plain rule, written out like oracle_topk_kk). */
int oracle_topk_kkk(const float* k1, const float* k2, const float* k3, uint64_t n, uint32_t k,
                    int order1, int order2, int order3, float* out_k1, float* out_k2,
                    float* out_k3, int64_t* out_idx) {
    if (!k1 || !k2 || !k3 || n == 0 || k == 0 || k > n) return -1;
    for (int o : {order1, order2, order3})
        if (o != 0 && o != 1) return -1;
    struct Row {
        uint64_t c1, c2, c3, idx;
    };
    std::vector<Row> v(n);
    for (uint64_t i = 0; i < n; ++i) {
        v[i].c1 = code_of(DT_F32, k1, i, order1);
        v[i].c2 = code_of(DT_F32, k2, i, order2);
        v[i].c3 = code_of(DT_F32, k3, i, order3);
        v[i].idx = i;
    }
    auto lex_better = [](const Row& a, const Row& b) {
        if (a.c1 != b.c1) return a.c1 > b.c1;
        if (a.c2 != b.c2) return a.c2 > b.c2;
        if (a.c3 != b.c3) return a.c3 > b.c3;
        return a.idx < b.idx;
    };
    std::partial_sort(v.begin(), v.begin() + k, v.end(), lex_better);
    for (uint32_t j = 0; j < k; ++j) {
        const uint64_t r = v[j].idx;
        if (out_idx) out_idx[j] = static_cast<int64_t>(r);
        if (out_k1) std::memcpy(out_k1 + j, k1 + r, 4);
        if (out_k2) std::memcpy(out_k2 + j, k2 + r, 4);
        if (out_k3) std::memcpy(out_k3 + j, k3 + r, 4);
    }
    return 0;
}

/* Order code of each key (exposed so tests can pin the code map itself against
 * IEEE-754 facts and against library sorts). */
void oracle_codes(int dtype, const void* keys, uint64_t n, int order, uint64_t* out) {
    for (uint64_t i = 0; i < n; ++i) out[i] = code_of(dtype, keys, i, order);
}

int oracle_threads(void) { return host_threads(0); }

}  // extern "C"
