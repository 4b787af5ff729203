// radix.cu -- radix-select top-k launch sequence (radix.cuh), the paper's selection-
// based alternative, for the cost-model comparison.
#include <cuda_runtime.h>

#include "dispatch.h"
#include "radix.cuh"

namespace topk {
namespace {

template <class Key, bool MIN>
cudaError_t radix_seq(const RadixParams& p, cudaStream_t st) {
    using C = typename CodeOf<typename KeyTraits<Key>::E>::C;
    static std::atomic<uint64_t> attr{0};  // per device (dispatch.h)
    const cudaError_t e = smem_attr_once(radix_final<Key, MIN>, static_cast<int>(kMergeSmem), attr);
    if (e != cudaSuccess) return e;
    const int G = static_cast<int>(p.G);
    radix_hist<Key, MIN, true><<<G, kHistNT, 0, st>>>(p);
    radix_choose<C, true><<<1, kRadixBins, 0, st>>>(p);
    radix_scatter<Key, MIN><<<G, kRadixNT, 0, st>>>(p);
    for (int d = 1; d < static_cast<int>(sizeof(C)); ++d) {  // the remaining digits
        radix_hist<Key, MIN, false><<<G, kHistNT, 0, st>>>(p);
        radix_choose<C, false><<<1, kRadixBins, 0, st>>>(p);
        radix_scatter<Key, MIN><<<G, kRadixNT, 0, st>>>(p);
    }
    radix_collect<C><<<G, kRadixNT, 0, st>>>(p);
    radix_emit<Key, MIN><<<G, kRadixNT, 0, st>>>(p);
    radix_final<Key, MIN><<<1, kMergeNT, kMergeSmem, st>>>(p);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_radix(int key, bool min_order, const RadixParams& p, cudaStream_t st,
                         int* launches) {
    const int nd = key == kKeyF64 ? 8 : 4;
    *launches = 3 * nd + 3;
    switch (key) {
        case kKeyF32: return min_order ? radix_seq<float, true>(p, st) : radix_seq<float, false>(p, st);
        case kKeyU32:
            return min_order ? radix_seq<uint32_t, true>(p, st) : radix_seq<uint32_t, false>(p, st);
        case kKeyF64: return min_order ? radix_seq<double, true>(p, st) : radix_seq<double, false>(p, st);
    }
    return cudaErrorInvalidValue;
}

size_t radix_workspace_bytes(int key, uint32_t G, uint32_t k, uint32_t cap) {
    return key == kKeyF64 ? radix_ws_bytes<uint64_t>(G, k, cap) : radix_ws_bytes<uint32_t>(G, k, cap);
}

}  // namespace topk
