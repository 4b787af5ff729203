// select_inst.cuh -- body of one generated translation unit (build/gen/, written by
// _build.py): ONE select_kernel instantiation plus its launcher and debug accessor.
// One kernel per TU keeps ptxas' inlining decisions those of the kernel alone: when
// several instantiations share a TU, the shared flush / network templates stop being
// inlined (calls + local-memory spills in the streaming loop, measured 1.6x slower).
// Defines before inclusion: TOPK_INST_KEY, TOPK_INST_MIN, TOPK_INST_FILTER,
// TOPK_INST_Q, TOPK_INST_FN (function name).
#pragma once
#include <atomic>

#include "dispatch.h"
#include "select.cuh"

#define TOPK_CAT2(a, b) a##b
#define TOPK_CAT(a, b) TOPK_CAT2(a, b)

namespace topk {

cudaError_t TOPK_INST_FN(const SelectParams& p, int grid, cudaStream_t st) {
    using Key = TOPK_INST_KEY;
    constexpr bool MIN = TOPK_INST_MIN, FILTER = TOPK_INST_FILTER;
    constexpr int Q = TOPK_INST_Q;
    static std::atomic<uint64_t> attr_set{0};  // per device (dispatch.h)
    const size_t smem = select_smem_bytes<Key, Q>();
    const cudaError_t e =
        smem_attr_once(select_kernel<Key, MIN, FILTER, Q>, static_cast<int>(smem), attr_set);
    if (e != cudaSuccess) return e;
    select_kernel<Key, MIN, FILTER, Q><<<grid, kNT, smem, st>>>(p);
    return cudaGetLastError();
}

// This TU's copy of the debug globals (select.cuh g_stats, g_trace, c_dbg, c_trace_on).
int TOPK_CAT(TOPK_INST_FN, _debug)(int op, void* host, int arg) {
#ifndef TOPK_DEBUG
    (void)op;
    (void)host;
    (void)arg;
    return -1;  // debug globals exist only in -DTOPK_DEBUG builds
#else
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
            return cudaMemcpyToSymbol(c_dbg_sym, &arg, sizeof(int)) == cudaSuccess ? 0 : -1;
        case kDbgTraceRead:  // host: u64[kTraceCtas][kTraceLen]
            return cudaMemcpyFromSymbol(host, g_trace, sizeof(g_trace)) == cudaSuccess ? 0 : -1;
        case kDbgTraceSet: {  // clear, then enable (arg = 1) or disable
            static unsigned long long zero[kTraceCtas][kTraceLen];
            if (cudaMemcpyToSymbol(g_trace, zero, sizeof(zero)) != cudaSuccess) return -1;
            return cudaMemcpyToSymbol(c_trace_on, &arg, sizeof(int)) == cudaSuccess ? 0 : -1;
        }
    }
    return -1;
#endif
}

}  // namespace topk
