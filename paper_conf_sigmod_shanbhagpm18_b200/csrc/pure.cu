// pure.cu -- instantiations and launcher of the pure-mode kernel (pure.cuh): 32-bit keys,
// max / min order, K = 2^L for L = 0 .. 5 (keys-only network) and 6 .. 8 (entries).
#include <cuda_runtime.h>

#include "dispatch.h"
#include "pure.cuh"

namespace topk {
namespace {

template <class Key, bool MIN, int L>
cudaError_t launch_pure_l(const PureParams& p, int grid, cudaStream_t st) {
    static std::atomic<uint64_t> attr{0};  // per device (dispatch.h)
    const cudaError_t e =
        smem_attr_once(pure_kernel<Key, MIN, L>, static_cast<int>(kPureSmem), attr);
    if (e != cudaSuccess) return e;
    pure_kernel<Key, MIN, L><<<grid, kPureNT, kPureSmem, st>>>(p);
    return cudaGetLastError();
}

template <class Key, bool MIN, int L>
cudaError_t launch_pure64_l(const PureParams& p, int grid, cudaStream_t st) {
    static std::atomic<uint64_t> attr{0};  // per device (dispatch.h)
    const cudaError_t e =
        smem_attr_once(pure64_kernel<Key, MIN, L>, static_cast<int>(kPureSmem), attr);
    if (e != cudaSuccess) return e;
    pure64_kernel<Key, MIN, L><<<grid, kPureNT, kPureSmem, st>>>(p);
    return cudaGetLastError();
}

template <class Key, bool MIN>
cudaError_t launch_pure_k(const PureParams& p, int grid, cudaStream_t st) {
    switch (p.L) {
        case 0: return launch_pure_l<Key, MIN, 0>(p, grid, st);
        case 1: return launch_pure_l<Key, MIN, 1>(p, grid, st);
        case 2: return launch_pure_l<Key, MIN, 2>(p, grid, st);
        case 3: return launch_pure_l<Key, MIN, 3>(p, grid, st);
        case 4: return launch_pure_l<Key, MIN, 4>(p, grid, st);
        case 5: return launch_pure_l<Key, MIN, 5>(p, grid, st);
        case 6: return launch_pure64_l<Key, MIN, 6>(p, grid, st);
        case 7: return launch_pure64_l<Key, MIN, 7>(p, grid, st);
        case 8: return launch_pure64_l<Key, MIN, 8>(p, grid, st);
    }
    return cudaErrorInvalidValue;
}

}  // namespace

cudaError_t launch_pure(int key, bool min_order, const PureParams& p, int grid, cudaStream_t st) {
    if (key == kKeyF32)
        return min_order ? launch_pure_k<float, true>(p, grid, st)
                         : launch_pure_k<float, false>(p, grid, st);
    if (key == kKeyU32)
        return min_order ? launch_pure_k<uint32_t, true>(p, grid, st)
                         : launch_pure_k<uint32_t, false>(p, grid, st);
    return cudaErrorInvalidValue;
}

}  // namespace topk
