// dispatch.h -- host-side interface between topk_api.cu and the per-key-type
// translation units that instantiate the streaming select kernel (select_f32.cu,
// select_u32.cu, select_f64.cu; the instantiations are compiled in parallel).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace topk {
struct SelectParams;

// Debug operations on one translation unit's device globals (select.cuh g_stats,
// g_trace, c_dbg, c_trace_on): each TU holds its own copy.
enum DebugOp { kDbgStatsAdd = 0, kDbgStatsReset = 1, kDbgFlags = 2, kDbgTraceRead = 3,
               kDbgTraceSet = 4 };

#define TOPK_DECLARE_SELECT_TU(NAME)                                                        \
    cudaError_t launch_select_##NAME(const SelectParams& p, int grid, bool min_order,       \
                                     bool filter, cudaStream_t st);                         \
    int debug_select_##NAME(int op, void* host, int arg);
TOPK_DECLARE_SELECT_TU(f32)
TOPK_DECLARE_SELECT_TU(u32)
TOPK_DECLARE_SELECT_TU(f64)
#undef TOPK_DECLARE_SELECT_TU

// Query forms (select.cuh QCfg: q = kQPred | kQRank bits; kQRank for f32 only).
#define TOPK_DECLARE_QUERY_TU(NAME)                                                         \
    cudaError_t launch_query_##NAME(const SelectParams& p, int grid, bool min_order, int q, \
                                    cudaStream_t st);                                       \
    int debug_query_##NAME(int op, void* host, int arg);
TOPK_DECLARE_QUERY_TU(f32)
TOPK_DECLARE_QUERY_TU(u32)
TOPK_DECLARE_QUERY_TU(f64)
TOPK_DECLARE_QUERY_TU(kk)
#undef TOPK_DECLARE_QUERY_TU

}  // namespace topk
