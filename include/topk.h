/*
 * include/topk.h -- C ABI of the B200-native bitonic top-k library (libtopk_b200.so).
 *
 * The operation (PAPER.md = /root/reference/PAPER.md, "P:<line>"):
 *   "find the top-k items, i.e., the largest or smallest ... according to some sort
 *   order (implemented via LIMIT or ORDER BY expressions in SQL)"  -- P:16 (Abstract);
 *   "finding the highest (or lowest) k of n tuples given a ranking function" -- P:32 (§1).
 * The method is the paper's bitonic top-k (§3.2; Alg. 4): local
 * sort into k-runs, merge of run pairs (keep the better element of each pair), rebuild
 * of the resulting bitonic k-sequences, repeated until k remain.  Key types follow the
 * paper's evaluation: float, unsigned int, double; key + value
 * by passing the tuple id around and assembling at the end.
 *
 * Result definition (readings R1-R5; the paper is silent on these):
 *   - total order: code(key) descending, then source index ascending (ties -> lowest
 *     index).  code(): NaN (any sign/payload) ranks above +inf and all NaNs tie; -0 and
 *     +0 tie; TOPK_SMALLEST reverses the key order but keeps "lowest index first".
 *   - out[0..k) is best first; out_keys[j] is bit-identical to keys[out_idx[j] - base].
 *   - any 1 <= k <= min(n, 2048) (k need not be a power of two; the paper evaluates
 *     1..1024, and its shared-memory form holds k <= 2048).
 *
 * Conventions for every call below:
 *   - Pointers named keys/payload/out_* and ws are DEVICE pointers (cudaMalloc or
 *     equivalent), except in topk_select_host where h_* are HOST pointers.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     All work is enqueued asynchronously on it; nothing synchronises the host.
 *   - Layout: 1-D contiguous arrays.  keys must be aligned to sizeof(key); 16-byte
 *     alignment is NOT required (the unaligned head/tail is peeled).  Outputs: out_keys
 *     [k] of the key type, out_idx [k] int64, out_payload [k] uint32; any may be NULL.
 *   - Ownership: the caller owns every buffer; the library never allocates device
 *     memory, never frees, and retains no pointer after the call returns.  Buffers must
 *     stay valid until the stream reaches the enqueued work.
 *   - Workspace: `ws` of at least topk_workspace_bytes(...) bytes, 256-byte aligned,
 *     zero-filled before its FIRST use (topk_workspace_init); every call leaves its
 *     control words zeroed again (the candidate area is scratch), so it needs no
 *     re-initialisation between calls.  One workspace must not be used by two calls concurrently;
 *     calls with distinct workspaces are re-entrant.
 *   - Errors: argument errors are returned synchronously and nothing is enqueued;
 *     launch failures return TOPK_ERR_CUDA; asynchronous faults surface at the caller's
 *     next synchronisation of `stream`.
 */
#ifndef TOPK_B200_H
#define TOPK_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define TOPK_ABI_VERSION 1
#define TOPK_MAX_K 2048

typedef enum {
    TOPK_OK = 0,
    TOPK_ERR_INVALID_ARG = 1, /* NULL input, k == 0, k > n, k > 2048, bad enum, alias  */
    TOPK_ERR_UNSUPPORTED = 2, /* device is not sm_100 (B200)                          */
    TOPK_ERR_WORKSPACE = 3,   /* ws NULL, too small or misaligned                      */
    TOPK_ERR_CUDA = 4,        /* a CUDA runtime call or kernel launch failed           */
    TOPK_ERR_NCCL = 5         /* an NCCL call failed (sharded entry points)            */
} topk_status_t;

typedef enum {
    TOPK_LARGEST = 0, /* ORDER BY key DESC LIMIT k */
    TOPK_SMALLEST = 1 /* ORDER BY key ASC  LIMIT k */
} topk_order_t;

typedef enum { TOPK_F32 = 0, TOPK_U32 = 1, TOPK_F64 = 2 } topk_dtype_t;

typedef enum {
    /* Default.  The streaming pass keeps a key only if it can still be in the top-k
     * (the paper's §5 "buffer filler", with the predicate "better than the
     * current k-th best"); survivors run through local sort / merge / rebuild.
     * Result identical to TOPK_MODE_PURE. */
    TOPK_MODE_FILTER = 0,
    /* The paper's pure method: every key goes through local sort, merge and rebuild
     * (SortReducer P:179-180).  Data-independent work. */
    TOPK_MODE_PURE = 1
} topk_mode_t;

/* Workspace bytes needed by topk_select / topk_* for (dtype, n, k) on the current
 * device.  Returns 0 if the arguments are invalid.  O(#SM * k * 12 B), < 4 MiB. */
size_t topk_workspace_bytes(topk_dtype_t dtype, uint64_t n, uint32_t k);

/* Zero-fill a workspace (enqueued on `stream`).  Needed once before first use. */
topk_status_t topk_workspace_init(void* ws, size_t ws_bytes, void* stream);

/* General entry point: top-k of keys[0..n) whose global row ids are base + i.
 *   dtype     TOPK_F32 (float), TOPK_U32 (uint32_t) or TOPK_F64 (double) keys.
 *   payload   optional uint32 column [n] gathered into out_payload; may be NULL.
 *   base      added to every output index (shard offset, §8(e)); 0 for a plain call.
 *   mode      TOPK_MODE_FILTER (default) or TOPK_MODE_PURE; same result.
 *   out_idx   receives base + i of each winner (int64). */
topk_status_t topk_select(topk_dtype_t dtype, const void* keys, const uint32_t* payload,
                          uint64_t n, uint64_t base, uint32_t k, topk_order_t order,
                          topk_mode_t mode, void* out_keys, uint32_t* out_payload,
                          int64_t* out_idx, void* ws, size_t ws_bytes, void* stream);

/* Typed conveniences (base = 0, mode = TOPK_MODE_FILTER). */
topk_status_t topk_f32(const float* keys, uint64_t n, uint32_t k, topk_order_t order,
                       float* out_keys, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream);
topk_status_t topk_u32(const uint32_t* keys, uint64_t n, uint32_t k, topk_order_t order,
                       uint32_t* out_keys, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream);
topk_status_t topk_f64(const double* keys, uint64_t n, uint32_t k, topk_order_t order,
                       double* out_keys, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream);
/* Key + payload: "ORDER BY key DESC LIMIT k" returning the 32-bit row id column. */
topk_status_t topk_u32_kv(const uint32_t* keys, const uint32_t* payload, uint64_t n,
                          uint32_t k, topk_order_t order, uint32_t* out_keys,
                          uint32_t* out_payload, int64_t* out_idx, void* ws,
                          size_t ws_bytes, void* stream);
topk_status_t topk_f64_kv(const double* keys, const uint32_t* payload, uint64_t n,
                          uint32_t k, topk_order_t order, double* out_keys,
                          uint32_t* out_payload, int64_t* out_idx, void* ws,
                          size_t ws_bytes, void* stream);

/* ---- Query form: the paper's §5 database integration ----
 *   SELECT row WHERE pred(row) ORDER BY f(row) DESC|ASC LIMIT k
 * "Fusing with filter": the predicate runs inside the streaming pass as the
 * FusedSortReducer's buffer filler -- a row enters the shared-memory buffer only if it
 * matches (and can still be in the top-k); nothing filtered is written to memory.
 * "Custom ranking function": f(A1, A2) is evaluated inside the same pass
 * instead of a separate projection.  Queries 1-3 of §6.8 have this shape.
 *   pred   NULL (no WHERE) or a topk_pred_t:
 *            TOPK_PRED_RANGE  lo <= col[i] < hi            ("tweet_time < X")
 *            TOPK_PRED_IN     col[i] < 64 and bit col[i] of in_mask set -- an IN list
 *                             over a dictionary-coded column ("lang='en' OR lang='es'",
 *                             P:300)
 *          col is a DEVICE uint32 column [n].
 *   rank_b NULL: f = keys[i] (dtype F32 / U32 / F64).  Otherwise (dtype F32 only) the
 *          ranking function f = keys[i] + rank_w * rank_b[i], the product and the sum
 *          each rounded to nearest float ("retweet_count + 0.5 * likes_count");
 *          rank_b is a DEVICE float column [n].
 *   Result: out_keys[j] = f of the j-th best matching row (best first, ties to the lowest
 *   row id, the order of topk_select), out_idx[j] its row id; when fewer than k rows
 *   match, rows j >= matches get out_idx = -1, out_keys = 0 bits, out_payload = 0.
 *   Layout: every column (keys, rank_b, pred->col, payload) 16-byte aligned, same n;
 *   1 <= k <= min(n, 2048); n <= 2^32 - 2.  Workspace: topk_workspace_bytes(dtype, n, k).
 *   Errors: TOPK_ERR_INVALID_ARG for a misaligned column, a bad predicate kind, rank_b
 *   with a non-F32 dtype, or neither pred nor rank_b (use topk_select). */
typedef enum { TOPK_PRED_RANGE = 1, TOPK_PRED_IN = 2 } topk_pred_kind_t;
typedef struct {
    topk_pred_kind_t kind;
    const uint32_t* col; /* DEVICE [n] */
    uint32_t lo, hi;     /* TOPK_PRED_RANGE */
    uint64_t in_mask;    /* TOPK_PRED_IN */
} topk_pred_t;
topk_status_t topk_query(topk_dtype_t dtype, const void* keys, const float* rank_b,
                         float rank_w, const topk_pred_t* pred, const uint32_t* payload,
                         uint64_t n, uint32_t k, topk_order_t order, void* out_keys,
                         uint32_t* out_payload, int64_t* out_idx, void* ws, size_t ws_bytes,
                         void* stream);

/* Compound keys -- "two keys + value (KKV)" (§6.6):
 *   SELECT row WHERE pred(row) ORDER BY keys1 [DESC|ASC], keys2 [DESC|ASC] LIMIT k
 * Lexicographic: keys1 decides (order1), keys2 breaks its ties (order2), then the lowest
 * row id; each column uses topk_select's float order (NaN greatest, -0 == +0).  The
 * value is the tuple id carried through the network and gathered at the end
 * ("pass around the tuple id and construct the full tuple at the end"):
 * out_idx, and out_payload = payload[row] if payload is given.  Both key columns stream
 * through the same single pass (8 bytes per row; 12 with a predicate).
 *   keys1, keys2  DEVICE float [n], 16-byte aligned; pred / payload as topk_query.
 *   out_keys1/2   DEVICE float [k] (either may be NULL); rows beyond the matches of a
 *                 predicate get out_idx = -1 and zero bits.
 *   ws            topk_workspace_bytes(TOPK_F64, n, k) bytes (12-byte entries).
 *   1 <= k <= min(n, 2048); n <= 2^32 - 2. */
topk_status_t topk_kk(const float* keys1, const float* keys2, const topk_pred_t* pred,
                      const uint32_t* payload, uint64_t n, uint32_t k, topk_order_t order1,
                      topk_order_t order2, float* out_keys1, float* out_keys2,
                      uint32_t* out_payload, int64_t* out_idx, void* ws, size_t ws_bytes,
                      void* stream);

/* Three compound keys -- "three keys + value (KKKV)" (§6.6): as topk_kk with
 * a third float column keys3 (order3) breaking the remaining ties; 12 bytes streamed per
 * row (16 with a predicate).  ws: topk_workspace_bytes(TOPK_F64, n, k) bytes. */
topk_status_t topk_kkk(const float* keys1, const float* keys2, const float* keys3,
                       const topk_pred_t* pred, const uint32_t* payload, uint64_t n, uint32_t k,
                       topk_order_t order1, topk_order_t order2, topk_order_t order3,
                       float* out_keys1, float* out_keys2, float* out_keys3,
                       uint32_t* out_payload, int64_t* out_idx, void* ws, size_t ws_bytes,
                       void* stream);

/* Radix-select top-k: the paper's selection-based method (§2.3 "Radix Select", P:93;
 * §4.2), the comparison point of its evaluation ("Radix Select for
 * larger K") and of its cost model (§7.1).  Same result as topk_select
 * (R1-R5: identical values, rows and order).  MSD passes over 8-bit digits of
 * the order code (4 for 32-bit keys, 8 for f64): histogram -> prefix sum -> the bucket
 * holding the k-th best; the bucket is written once, at the first digit where it fits
 * the workspace, with every entry above it; later digits read only the bucket; ties
 * at the k-th code resolve to the lowest rows (a further input pass when the ties do
 * not fit).  At least two reads of the input (histogram + bucket pass), against one
 * for topk_select -- the reason the bench's dispatch keeps bitonic top-k on B200.
 *   keys      DEVICE array [n] of the dtype; n <= 2^32 - 2.
 *   ws        topk_radix_workspace_bytes(dtype, n, k) bytes (O(n / 16 * entry): the
 *             bucket; cf. "selection-based methods require an additional buffer",
 *             P:209), 256-byte aligned, zero-filled before first use; left zeroed.
 *   Enqueues 15 (32-bit keys) or 27 (f64) kernels on `stream`, no host sync. */
size_t topk_radix_workspace_bytes(topk_dtype_t dtype, uint64_t n, uint32_t k);
topk_status_t topk_radix(topk_dtype_t dtype, const void* keys, uint64_t n, uint32_t k,
                         topk_order_t order, void* out_keys, int64_t* out_idx, void* ws,
                         size_t ws_bytes, void* stream);

/* Top-k of keys in HOST memory (pinned memory strongly recommended): the input is
 * streamed to the device in chunks of `chunk_keys` keys through a double-buffered
 * staging area inside `ws`; each chunk's top-k runs as soon as it has landed, so the
 * copies overlap the reductive pass -- "the reductive nature of top-k queries makes it
 * trivial to process the data in memory-size chunks and overlap computation with
 * transfer" -- and the chunk results are merged (topk_merge).  h_out_keys /
 * h_out_idx are HOST pointers, written when `stream` reaches the end of the call.
 *   chunk_keys  multiple of 4, >= 4096; ceil(n / chunk_keys) * k <= 65536.
 *   ws          DEVICE workspace of topk_host_workspace_bytes(dtype, n, k, chunk_keys).
 * Uses one library-owned copy stream per device (not re-entrant across host threads). */
size_t topk_host_workspace_bytes(topk_dtype_t dtype, uint64_t n, uint32_t k,
                                 uint64_t chunk_keys);
topk_status_t topk_select_host(topk_dtype_t dtype, const void* h_keys, uint64_t n, uint32_t k,
                               topk_order_t order, void* h_out_keys, int64_t* h_out_idx,
                               uint64_t chunk_keys, void* ws, size_t ws_bytes, void* stream);

/* Global step of the partitioned top-k (§1, App. C; multi-GPU §8(e)):
 * the exact top-k of `runs` candidate lists of `run_len` entries each, laid out
 * back to back: cand_keys[runs*run_len] (key type), cand_idx[runs*run_len] int64
 * global row ids (the tie-break), cand_payload optional.  Entries may be in any order;
 * duplicated (key, idx) entries are not allowed.  1 <= k <= min(runs*run_len, 2048),
 * runs*run_len <= 65536.  Single-CTA local sort + merge + rebuild network (in chunks of
 * 4096 entries next to the running top-k); ws as topk_merge_workspace_bytes (unused). */
size_t topk_merge_workspace_bytes(topk_dtype_t dtype, uint32_t runs, uint32_t run_len,
                                  uint32_t k);
topk_status_t topk_merge(topk_dtype_t dtype, const void* cand_keys, const int64_t* cand_idx,
                         const uint32_t* cand_payload, uint32_t runs, uint32_t run_len,
                         uint32_t k, topk_order_t order, void* out_keys,
                         uint32_t* out_payload, int64_t* out_idx, void* ws,
                         size_t ws_bytes, void* stream);

/* topk_merge for candidates whose every run is sorted best first -- the order every
 * topk_select / topk_* result has (the multi-GPU all-gather, chunked inputs): the kernel
 * skips the local sort and runs log2(runs) rounds of the paper's merge + rebuild over
 * the runs (run 2i as is, run 2i+1 reversed: each pair is one bitonic sequence, P:150;
 * Alg. 4).  Same arguments and result as topk_merge; a run's entries past position
 * next_pow2(k) are never read.  Passing unsorted runs gives an unspecified result. */
topk_status_t topk_merge_sorted(topk_dtype_t dtype, const void* cand_keys,
                                const int64_t* cand_idx, const uint32_t* cand_payload,
                                uint32_t runs, uint32_t run_len, uint32_t k, topk_order_t order,
                                void* out_keys, uint32_t* out_payload, int64_t* out_idx,
                                void* ws, size_t ws_bytes, void* stream);

/* ---- Multi-GPU: the partitioned top-k (§1 "per-partition top-k ... global top-k
 * from the m per-partition heaps"; App. C "combined in a final global step") ----
 * One process (or thread) per GPU; rank r holds the global rows [base, base + n_local)
 * of the input.  topk_select_sharded runs, enqueued on `stream`:
 *   (1) the local top-k of keys[0 .. n_local) (topk_select, ids base + i),
 *   (2) ncclAllGather of the k (key, int64 id[, uint32 payload]) candidates of every
 *       rank over `comm` (NVLink / NVSwitch),
 *   (3) topk_merge of the nranks * k candidates -- the exact global top-k, ties to the
 *       lowest GLOBAL id, identical on every rank.
 * Collective: every rank of `comm` must call it with the same k and order (and all with
 * or all without payload).  n_local >= k on every rank; nranks * k <= 65536.
 * comm is an ncclComm_t (as void*) -- made with topk_nccl_comm_init, or any NCCL
 * communicator of the same NCCL library.  ws: DEVICE workspace of
 * topk_sharded_workspace_bytes(...) bytes, 256-byte aligned, zero-filled before first
 * use (topk_workspace_init).  Outputs are DEVICE pointers (k entries, any may be NULL).
 * NCCL is loaded at run time (libnccl.so.2; the copy already in the process if any):
 * TOPK_ERR_UNSUPPORTED if it cannot be found, TOPK_ERR_NCCL if a call fails. */
#define TOPK_NCCL_UNIQUE_ID_BYTES 128
/* ncclGetUniqueId into id[128] (host memory), to be broadcast to every rank. */
topk_status_t topk_nccl_unique_id(void* id);
/* ncclCommInitRank(comm, nranks, id, rank); *comm receives the ncclComm_t.  The calling
 * thread's current CUDA device is the rank's device.  Collective over the ranks. */
topk_status_t topk_nccl_comm_init(const void* id, int nranks, int rank, void** comm);
topk_status_t topk_nccl_comm_destroy(void* comm);
size_t topk_sharded_workspace_bytes(topk_dtype_t dtype, uint64_t n_local, uint32_t k,
                                    int nranks);
topk_status_t topk_select_sharded(topk_dtype_t dtype, const void* keys, const uint32_t* payload,
                                  uint64_t n_local, uint64_t base, uint32_t k,
                                  topk_order_t order, void* out_keys, uint32_t* out_payload,
                                  int64_t* out_idx, void* comm, void* ws, size_t ws_bytes,
                                  void* stream);
/* f32 convenience. */
topk_status_t topk_f32_sharded(const float* keys, uint64_t n_local, uint64_t base, uint32_t k,
                               topk_order_t order, float* out_keys, int64_t* out_idx, void* comm,
                               void* ws, size_t ws_bytes, void* stream);

/* Read-bandwidth probe (the paper's "Memory Bandwidth" line: the time to read
 * the data once, a lower bound for any top-k): reads `bytes` (multiple of 16, 16-byte
 * aligned) at `data` once.  method 0: 128-bit non-coherent loads, `grid` CTAs of 512
 * threads (0 = 4 per SM); method 1: the top-k pass's TMA ring (`tile` bytes x `stages`,
 * one CTA per SM).  `sink` is a device uint32 (scratch).  Enqueued on `stream`. */
topk_status_t topk_probe_read(const void* data, size_t bytes, int method, int grid, int tile,
                              int stages, uint32_t* sink, void* stream);

/* Number of kernels this library has launched in this process (for the bench's
 * "gpu_launches" count).  Thread-safe, monotone. */
uint64_t topk_launch_count(void);

/* Static description of a status code. */
const char* topk_status_string(topk_status_t s);

/* TOPK_ABI_VERSION of the loaded library. */
int topk_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TOPK_B200_H */
