// select_tu.cuh -- body of one select translation unit: instantiates select_kernel for
// one key type (both orders, filter and pure modes) and the TU's debug accessors.
// Include after defining TOPK_TU_KEY (the key type) and TOPK_TU_NAME (f32 | u32 | f64).
// With TOPK_TU_QUERY defined the TU instead instantiates the query forms (WHERE
// predicate; for f32 also the ranking function), as launch_query_<NAME> /
// debug_query_<NAME>.
#pragma once
#include <atomic>

#include "dispatch.h"
#include "select.cuh"

#define TOPK_CAT2(a, b) a##b
#define TOPK_CAT(a, b) TOPK_CAT2(a, b)

namespace topk {
namespace {

template <class Key, bool MIN, bool FILTER, int Q = 0>
cudaError_t launch_one(const SelectParams& p, int grid, cudaStream_t st) {
    static std::atomic<bool> attr_set{false};  // per instantiation (idempotent)
    const size_t smem = select_smem_bytes<Key>();
    if (!attr_set.load(std::memory_order_relaxed)) {
        cudaError_t e = cudaFuncSetAttribute(select_kernel<Key, MIN, FILTER, Q>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             static_cast<int>(smem));
        if (e != cudaSuccess) return e;
        attr_set.store(true, std::memory_order_relaxed);
    }
    select_kernel<Key, MIN, FILTER, Q><<<grid, kNT, smem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace

#ifndef TOPK_TU_QUERY
#define TOPK_TU_KIND select_
cudaError_t TOPK_CAT(launch_select_, TOPK_TU_NAME)(const SelectParams& p, int grid,
                                                   bool min_order, bool filter,
                                                   cudaStream_t st) {
    using Key = TOPK_TU_KEY;
    if (min_order)
        return filter ? launch_one<Key, true, true>(p, grid, st)
                      : launch_one<Key, true, false>(p, grid, st);
    return filter ? launch_one<Key, false, true>(p, grid, st)
                  : launch_one<Key, false, false>(p, grid, st);
}
#else
#define TOPK_TU_KIND query_
cudaError_t TOPK_CAT(launch_query_, TOPK_TU_NAME)(const SelectParams& p, int grid,
                                                  bool min_order, int q, cudaStream_t st) {
    using Key = TOPK_TU_KEY;
    if constexpr (std::is_same<Key, KK32>::value) {  // compound keys (+ optional WHERE)
        switch (q) {
            case kQKey2:
                return min_order ? launch_one<Key, true, true, kQKey2>(p, grid, st)
                                 : launch_one<Key, false, true, kQKey2>(p, grid, st);
            case kQKey2 | kQPred:
                return min_order ? launch_one<Key, true, true, kQKey2 | kQPred>(p, grid, st)
                                 : launch_one<Key, false, true, kQKey2 | kQPred>(p, grid, st);
        }
        return cudaErrorInvalidValue;
    } else if constexpr (std::is_same<Key, float>::value) {
        switch (q) {
            case kQPred:
                return min_order ? launch_one<Key, true, true, kQPred>(p, grid, st)
                                 : launch_one<Key, false, true, kQPred>(p, grid, st);
            case kQRank:
                return min_order ? launch_one<Key, true, true, kQRank>(p, grid, st)
                                 : launch_one<Key, false, true, kQRank>(p, grid, st);
            case kQPred | kQRank:
                return min_order ? launch_one<Key, true, true, kQPred | kQRank>(p, grid, st)
                                 : launch_one<Key, false, true, kQPred | kQRank>(p, grid, st);
        }
        return cudaErrorInvalidValue;
    } else {
        if (q != kQPred) return cudaErrorInvalidValue;
        return min_order ? launch_one<Key, true, true, kQPred>(p, grid, st)
                         : launch_one<Key, false, true, kQPred>(p, grid, st);
    }
}
#endif

int TOPK_CAT(TOPK_CAT(debug_, TOPK_TU_KIND), TOPK_TU_NAME)(int op, void* host, int arg) {
    switch (op) {
        case kDbgStatsAdd: {  // host: u64[8], accumulated
            unsigned long long v[8];
            if (cudaMemcpyFromSymbol(v, g_stats, sizeof(v)) != cudaSuccess) return -1;
            uint64_t* h = static_cast<uint64_t*>(host);
            for (int i = 0; i < 8; ++i) h[i] += v[i];
            return 0;
        }
        case kDbgStatsReset: {
            unsigned long long z[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            return cudaMemcpyToSymbol(g_stats, z, sizeof(z)) == cudaSuccess ? 0 : -1;
        }
        case kDbgFlags:
            return cudaMemcpyToSymbol(c_dbg, &arg, sizeof(int)) == cudaSuccess ? 0 : -1;
        case kDbgTraceRead:  // host: u64[kTraceCtas][kTraceLen]
            return cudaMemcpyFromSymbol(host, g_trace, sizeof(g_trace)) == cudaSuccess ? 0 : -1;
        case kDbgTraceSet: {  // clear, then enable (arg = 1) or disable
            static unsigned long long zero[kTraceCtas][kTraceLen];
            if (cudaMemcpyToSymbol(g_trace, zero, sizeof(zero)) != cudaSuccess) return -1;
            return cudaMemcpyToSymbol(c_trace_on, &arg, sizeof(int)) == cudaSuccess ? 0 : -1;
        }
    }
    return -1;
}

}  // namespace topk
