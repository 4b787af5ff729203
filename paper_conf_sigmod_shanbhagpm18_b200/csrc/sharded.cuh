// sharded.cuh -- the multi-GPU entry of the C ABI (included by topk_api.cu).
//
// The paper's partitioned top-k: "each processor compute[s] a per-partition top-k and
// [the] global top-k [is computed] from the m per-partition heaps" (§1); "the top-k
// elements emitted by the individual core are combined in a final global step".
// One process per GPU: rank r holds global rows [base_r, base_r + n_local).
//   (1) local top-k of the shard (the select kernel, ids = base_r + i);
//   (2) ncclAllGather of the k (key, int64 id[, payload]) candidates of every rank
//       (NVLink 5 / NVSwitch; G * k entries, <= 8 * 1024 * 20 B -- latency bound);
//   (3) the merge kernel (local sort / merge / rebuild over the G sorted runs) -- exact
//       because ties break on the GLOBAL id, and identical on every rank.
// NCCL is resolved at run time (dlopen of libnccl.so.2, preferring the copy the process
// already loaded, e.g. PyTorch's), so the library has no link-time NCCL dependency;
// nccl.h supplies the types only.
#pragma once
#include <dlfcn.h>
#include <nccl.h>

#include <mutex>

namespace {

struct NcclApi {
    bool ok = false;
    ncclResult_t (*get_unique_id)(ncclUniqueId*) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    ncclResult_t (*comm_count)(const ncclComm_t, int*) = nullptr;
    ncclResult_t (*all_gather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t,
                               cudaStream_t) = nullptr;
    ncclResult_t (*group_start)() = nullptr;
    ncclResult_t (*group_end)() = nullptr;
};

NcclApi& nccl_api() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return;
        api.get_unique_id = reinterpret_cast<decltype(api.get_unique_id)>(dlsym(h, "ncclGetUniqueId"));
        api.comm_init_rank = reinterpret_cast<decltype(api.comm_init_rank)>(dlsym(h, "ncclCommInitRank"));
        api.comm_destroy = reinterpret_cast<decltype(api.comm_destroy)>(dlsym(h, "ncclCommDestroy"));
        api.comm_count = reinterpret_cast<decltype(api.comm_count)>(dlsym(h, "ncclCommCount"));
        api.all_gather = reinterpret_cast<decltype(api.all_gather)>(dlsym(h, "ncclAllGather"));
        api.group_start = reinterpret_cast<decltype(api.group_start)>(dlsym(h, "ncclGroupStart"));
        api.group_end = reinterpret_cast<decltype(api.group_end)>(dlsym(h, "ncclGroupEnd"));
        api.ok = api.get_unique_id && api.comm_init_rank && api.comm_destroy && api.comm_count &&
                 api.all_gather && api.group_start && api.group_end;
    });
    return api;
}

struct ShardLayout {
    size_t sel, lk, li, lp, lr, gk, gi, gp, gr, total;
};

ShardLayout shard_layout(topk_dtype_t dtype, uint64_t n_local, uint32_t k, int nranks) {
    ShardLayout L;
    L.sel = 0;
    const size_t sel_bytes = topk_workspace_bytes(dtype, n_local, k);
    const size_t ks = key_size(dtype);
    L.lk = align_up(sel_bytes, 256);
    L.li = L.lk + align_up(static_cast<size_t>(k) * ks, 256);
    L.lp = L.li + align_up(static_cast<size_t>(k) * 8, 256);
    L.lr = L.lp + align_up(static_cast<size_t>(k) * 4, 256);
    L.gk = L.lr + 256;
    L.gi = L.gk + align_up(static_cast<size_t>(nranks) * k * ks, 256);
    L.gp = L.gi + align_up(static_cast<size_t>(nranks) * k * 8, 256);
    L.gr = L.gp + align_up(static_cast<size_t>(nranks) * k * 4, 256);
    L.total = L.gr + align_up(static_cast<size_t>(nranks) * 16, 256);
    return L;
}

}  // namespace

extern "C" {

topk_status_t topk_nccl_unique_id(void* id) {
    if (!id) return TOPK_ERR_INVALID_ARG;
    NcclApi& a = nccl_api();
    if (!a.ok) return TOPK_ERR_UNSUPPORTED;
    ncclUniqueId u;
    if (a.get_unique_id(&u) != ncclSuccess) return TOPK_ERR_NCCL;
    std::memcpy(id, &u, sizeof(u));
    return TOPK_OK;
}

topk_status_t topk_nccl_comm_init(const void* id, int nranks, int rank, void** comm) {
    if (!id || !comm || nranks < 1 || rank < 0 || rank >= nranks) return TOPK_ERR_INVALID_ARG;
    NcclApi& a = nccl_api();
    if (!a.ok) return TOPK_ERR_UNSUPPORTED;
    ncclUniqueId u;
    std::memcpy(&u, id, sizeof(u));
    ncclComm_t c = nullptr;
    if (a.comm_init_rank(&c, nranks, u, rank) != ncclSuccess) return TOPK_ERR_NCCL;
    *comm = c;
    return TOPK_OK;
}

topk_status_t topk_nccl_comm_destroy(void* comm) {
    if (!comm) return TOPK_ERR_INVALID_ARG;
    NcclApi& a = nccl_api();
    if (!a.ok) return TOPK_ERR_UNSUPPORTED;
    return a.comm_destroy(static_cast<ncclComm_t>(comm)) == ncclSuccess ? TOPK_OK : TOPK_ERR_NCCL;
}

size_t topk_sharded_workspace_bytes(topk_dtype_t dtype, uint64_t n_local, uint32_t k,
                                    int nranks) {
    if (nranks < 1 || topk_workspace_bytes(dtype, n_local, k) == 0) return 0;
    if (static_cast<uint64_t>(nranks) * k > 65536) return 0;
    return shard_layout(dtype, n_local, k, nranks).total;
}

topk_status_t topk_select_sharded(topk_dtype_t dtype, const void* keys, const uint32_t* payload,
                                  uint64_t n_local, uint64_t base, uint32_t k,
                                  topk_order_t order, void* out_keys, uint32_t* out_payload,
                                  int64_t* out_idx, void* comm, void* ws, size_t ws_bytes,
                                  void* stream) {
    if (!valid_dtype(dtype) || !valid_order(order) || !keys || !comm) return TOPK_ERR_INVALID_ARG;
    if (k == 0 || k > TOPK_MAX_K || k > n_local) return TOPK_ERR_INVALID_ARG;
    if (out_payload && !payload) return TOPK_ERR_INVALID_ARG;
    NcclApi& a = nccl_api();
    if (!a.ok) return TOPK_ERR_UNSUPPORTED;
    int nranks = 0;
    if (a.comm_count(static_cast<ncclComm_t>(comm), &nranks) != ncclSuccess || nranks < 1)
        return TOPK_ERR_NCCL;
    if (static_cast<uint64_t>(nranks) * k > 65536) return TOPK_ERR_UNSUPPORTED;
    const ShardLayout L = shard_layout(dtype, n_local, k, nranks);
    if (!ws || ws_bytes < L.total || reinterpret_cast<uintptr_t>(ws) % 256) return TOPK_ERR_WORKSPACE;
    unsigned char* w = static_cast<unsigned char*>(ws);
    const size_t ks = key_size(dtype);
    // (1) local top-k with global ids
    topk_status_t s = topk_select(dtype, keys, payload, n_local, base, k, order, TOPK_MODE_FILTER,
                                  w + L.lk, payload ? reinterpret_cast<uint32_t*>(w + L.lp) : nullptr,
                                  reinterpret_cast<int64_t*>(w + L.li), w + L.sel, L.lk, stream);
    if (s != TOPK_OK) return s;
    // (2) all-gather the candidates of every rank, and every rank's row range (the merge
    // narrows its entries when the ranges increase rank by rank)
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const uint64_t range[2] = {base, n_local};  // pageable: staged at once, stream-ordered
    if (cudaMemcpyAsync(w + L.lr, range, sizeof(range), cudaMemcpyHostToDevice, st) != cudaSuccess)
        return TOPK_ERR_CUDA;
    ncclComm_t c = static_cast<ncclComm_t>(comm);
    if (a.group_start() != ncclSuccess) return TOPK_ERR_NCCL;
    ncclResult_t r = a.all_gather(w + L.lk, w + L.gk, k * ks, ncclUint8, c, st);
    if (r == ncclSuccess) r = a.all_gather(w + L.li, w + L.gi, k, ncclInt64, c, st);
    if (r == ncclSuccess && payload) r = a.all_gather(w + L.lp, w + L.gp, k, ncclUint32, c, st);
    if (r == ncclSuccess) r = a.all_gather(w + L.lr, w + L.gr, 2, ncclUint64, c, st);
    const ncclResult_t r2 = a.group_end();
    if (r != ncclSuccess || r2 != ncclSuccess) return TOPK_ERR_NCCL;
    // (3) the global step: exact top-k of the G sorted candidate runs
    return merge_total(dtype, w + L.gk, reinterpret_cast<const int64_t*>(w + L.gi),
                       payload ? reinterpret_cast<const uint32_t*>(w + L.gp) : nullptr,
                       static_cast<uint64_t>(nranks) * k, k, true, k, order, out_keys,
                       out_payload, out_idx, stream, false,
                       reinterpret_cast<const uint64_t*>(w + L.gr));
}

topk_status_t topk_f32_sharded(const float* keys, uint64_t n_local, uint64_t base, uint32_t k,
                               topk_order_t order, float* out_keys, int64_t* out_idx, void* comm,
                               void* ws, size_t ws_bytes, void* stream) {
    return topk_select_sharded(TOPK_F32, keys, nullptr, n_local, base, k, order, out_keys, nullptr,
                               out_idx, comm, ws, ws_bytes, stream);
}

}  // extern "C"
