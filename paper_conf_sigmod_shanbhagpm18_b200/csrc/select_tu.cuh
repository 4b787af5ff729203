// select_tu.cuh -- body of one select translation unit: instantiates select_kernel for
// one key type (both orders, filter and pure modes) and the TU's debug accessors.
// Include after defining TOPK_TU_KEY (the key type) and TOPK_TU_NAME (f32 | u32 | f64).
#pragma once
#include <atomic>

#include "dispatch.h"
#include "select.cuh"

#define TOPK_CAT2(a, b) a##b
#define TOPK_CAT(a, b) TOPK_CAT2(a, b)

namespace topk {
namespace {

template <class Key, bool MIN, bool FILTER>
cudaError_t launch_one(const SelectParams& p, int grid, cudaStream_t st) {
    static std::atomic<bool> attr_set{false};  // per instantiation (idempotent)
    const size_t smem = select_smem_bytes<Key>();
    if (!attr_set.load(std::memory_order_relaxed)) {
        cudaError_t e = cudaFuncSetAttribute(select_kernel<Key, MIN, FILTER>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             static_cast<int>(smem));
        if (e != cudaSuccess) return e;
        attr_set.store(true, std::memory_order_relaxed);
    }
    select_kernel<Key, MIN, FILTER><<<grid, kNT, smem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace

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

int TOPK_CAT(debug_select_, TOPK_TU_NAME)(int op, void* host, int arg) {
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
