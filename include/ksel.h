/*
 * ksel.h -- C ABI of libksel.so: B200-native (sm_100a) batched k-selection and
 * fused brute-force k-NN.
 *
 * Paper: Tang, Huang, Eyers, Mills, Guo, "Efficient Selection Algorithm for
 * Fast k-NN Search on GPU", IPDPS 2015.  Citations are PAPER.md line numbers.
 *
 * Common conventions
 * ------------------
 *  - All array pointers are CUDA DEVICE pointers owned by the caller (except
 *    the *_host entry points, documented below).  Arrays are dense row-major.
 *    Inputs are read-only; outputs are fully overwritten (all Q*k entries).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Every call is stream-ordered and asynchronous: it validates its
 *    arguments on the host, enqueues kernels and returns; it never
 *    synchronises the stream and allocates no device memory.
 *  - Order ("lexicographic (value, index)", readings R1-R5 in DESIGN.md):
 *    values compare as IEEE fp32 with -0.0 == +0.0, NaN greater than +Inf and
 *    all NaNs equal, denormals exact; equal values are ordered by the lower
 *    index.  Results are BIT-EXACT with the CPU oracle (oracle/).
 *  - Indices are int32, 0-based.
 *  - Thread-safe: no global mutable state except a lazily created, mutex-
 *    protected device-property cache and (host entry points only) per-device
 *    copy streams.
 *  - Errors: a nonzero ksel_status is returned; no exception crosses the ABI
 *    and nothing aborts.  Argument errors are detected before any launch.  A
 *    launch failure (cudaGetLastError after the launch) is KSEL_ERR_CUDA; the
 *    CUDA error itself is left in place (sticky errors are not cleared).
 */
#ifndef KSEL_H_
#define KSEL_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define KSEL_API __attribute__((visibility("default")))
#else
#define KSEL_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    KSEL_OK = 0,
    KSEL_ERR_INVALID_ARG = 1, /* null pointer, bad size, misalignment, aliasing */
    KSEL_ERR_UNSUPPORTED = 2, /* valid request outside this build's range (k > 1024) */
    KSEL_ERR_CUDA = 3,        /* a CUDA runtime call or kernel launch failed */
    KSEL_ERR_NO_DEVICE = 4,   /* no sm_100 device is current */
    KSEL_ERR_TIMEOUT = 5      /* a device-side flag wait gave up (ksel_device_status) */
} ksel_status;

#define KSEL_MAX_K 1024

/* ksel_select -- batched k-selection ("finding the k smallest
 * values from a given unordered list"; L19 Algorithm 1; L637 sorted output).
 *
 *   dist     [Q][N] fp32, device, 4-byte aligned (16-byte alignment of each row
 *            start is not required; unaligned heads/tails are handled).
 *   Q >= 1 rows, 1 <= N <= 2^31 - 1 columns, 1 <= k <= min(N, KSEL_MAX_K).
 *   out_val  [Q][k] fp32, device: out_val[q][t] has the same BITS as
 *            dist[q][out_idx[q][t]] (including -0.0 and NaN payloads).
 *   out_idx  [Q][k] int32, device.
 * out[q][0..k) = the k smallest pairs (dist[q][j], j) in lexicographic
 * (value, index) order, ascending.  Outputs must not overlap dist.
 * k > KSEL_MAX_K with k <= N returns KSEL_ERR_UNSUPPORTED. */
KSEL_API int ksel_select(const float* dist, int64_t Q, int64_t N, int k, float* out_val,
                int32_t* out_idx, void* stream);

/* ksel_select_ex -- ksel_select with a caller-provided device workspace, which
 * lets few long rows use the whole GPU (split rows): when Q is below
 * the SM count, every row is cut into S equal segments (S * Q <= #SMs, each
 * >= max(32768, 64 k') elements), each segment's top-k is selected by its own
 * CTA (row-global indices), and a second selection over each row's S*k
 * candidates merges them -- the divide-and-merge of PAPER.md L243 (ref. [18]);
 * ties there fall in index order, so the result is identical to ksel_select's.
 *   d_work  device workspace of >= ksel_select_workspace(Q, N, k) bytes (the
 *           segment lists), not overlapping the inputs/outputs; when that size
 *           is 0 (enough rows) or d_work is NULL, this is ksel_select.
 * Errors as ksel_select; a non-NULL workspace that is too small or overlaps ->
 * KSEL_ERR_INVALID_ARG. */
KSEL_API size_t ksel_select_workspace(int64_t Q, int64_t N, int k);
KSEL_API int ksel_select_ex(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx,
                            void* d_work, size_t work_bytes, void* stream);

/* ksel_select_config -- ksel_select with the kernel variant fixed (ablation /
 * tuning; same result bits for every variant):
 *   algo           KSEL_ALGO_AUTO (0), KSEL_ALGO_QUEUE (1): candidates merged into a
 *                  warp-register bitonic queue at every buffer flush (Merge Queue +
 *                  Buffered Search), KSEL_ALGO_POOL (2):
 *                  candidate pool narrowed by radix-histogram select (Hierarchical
 *                  Partition's discard-by-group, L221-L231, with value buckets),
 *                  KSEL_ALGO_RADIX (3): N <= 65536 only (else KSEL_ERR_UNSUPPORTED):
 *                  a cluster of <= 8 CTAs holds the row in registers and narrows
 *                  the exact k-th key by four 8-bit radix passes over all of it
 *                  (HP's value buckets, L225), then sorts the k selected pairs.
 *                  KSEL_ALGO_HIST (4): one CTA per row, a shared-memory pool narrowed
 *                  by range-adaptive radix histograms -- built into the experiments
 *                  library only (KSEL_BUILD_EXPERIMENTS=1); KSEL_ERR_UNSUPPORTED here.
 *   warps_per_row  0 = automatic, else 1, 2, 4 or 8 warps cooperating on each row
 *                  (ignored by KSEL_ALGO_RADIX).
 * Other arguments as ksel_select; invalid algo / warps_per_row -> INVALID_ARG. */
#define KSEL_ALGO_AUTO 0
#define KSEL_ALGO_QUEUE 1
#define KSEL_ALGO_POOL 2
#define KSEL_ALGO_RADIX 3
#define KSEL_ALGO_HIST 4
KSEL_API int ksel_select_config(const float* dist, int64_t Q, int64_t N, int k, float* out_val,
                                int32_t* out_idx, int algo, int warps_per_row, void* stream);

/* ksel_select_host -- the same operation on HOST buffers (the end-to-end entry
 * point a user without device memory calls).  h_dist [Q][N], h_out_val and
 * h_out_idx [Q][k] are host pointers (page-locked memory gives overlapped
 * copies; pageable memory works but serialises).  The library streams row
 * blocks host->device, selects, and copies results back, double-buffered
 * across two internal copy streams, using the caller's device workspace
 * `d_work` of `work_bytes` bytes (query the minimum with
 * ksel_select_host_workspace).  The copies start only after all work already
 * queued on `stream` (the workspace and the output buffers may still be in use
 * by it).  Returns after the results are in host memory (this call
 * synchronises; on an error it also waits for every copy it issued, so no
 * transfer touches the host buffers after it returns).  Same ordering /
 * bit-exactness as ksel_select. */
KSEL_API size_t ksel_select_host_workspace(int64_t N, int k);
KSEL_API int ksel_select_host(const float* h_dist, int64_t Q, int64_t N, int k, float* h_out_val,
                     int32_t* h_out_idx, void* d_work, size_t work_bytes, void* stream);

/* ksel_merge -- final merge of S per-shard candidate lists (divide-and-merge,
 * PAPER.md L243 ref. [18]; Merge Queue merging sorted levels, L41, L139).
 *   cand_val, cand_idx  [S][Q][kin], device.  For every (s, q) the list
 *            cand_*[s][q][0..kin) is sorted ascending in (value, index) order
 *            (exactly what ksel_select / knn_search emit).  Indices must be
 *            unique per query across all lists (e.g. global reference ids).
 *   1 <= S <= 64, 1 <= kin <= KSEL_MAX_K, 1 <= k <= min(S*kin, KSEL_MAX_K).
 *   out_val/out_idx [Q][k]: the k smallest pairs of the union, ascending;
 *            out_val keeps the candidates' bits.
 * Used after the NCCL all-gather of the row-sharded k-NN (S = world size). */
KSEL_API int ksel_merge(const float* cand_val, const int32_t* cand_idx, int64_t Q, int S, int kin, int k,
               float* out_val, int32_t* out_idx, void* stream);

/* knn_search -- brute-force k-NN: distance phase (Sec. II.A,
 * "the method of [3]" L243) fused with k-selection.
 *   ref   [N][D] fp32, query [Q][D] fp32, device, 4-byte aligned, row-major.
 *   1 <= D <= 256 (D > 256 -> KSEL_ERR_UNSUPPORTED); 1 <= k <= min(N, KSEL_MAX_K);
 *   N + idx_offset <= 2^31 - 1, idx_offset >= 0.
 *   out_dist [Q][k] fp32: squared L2 distance (no sqrt, reading R9) computed
 *            EXACTLY as the oracle does: (float) sum_t (q_t - r_t)^2 with the
 *            differences, squares and the index-ordered sum in double;
 *   out_idx  [Q][k] int32: idx_offset + reference row, ascending by
 *            (distance, index) -- bit-identical to the CPU oracle.
 *   d_work   device workspace of >= knn_search_workspace(N, Q, D, k) bytes
 *            (fp16 operand images, per-query candidate pools; queries are
 *            processed in chunks so that the pools stay below 2 GiB).
 * Method: a one-pass fp16 tcgen05 GEMM on centred operands scaled per tile by
 * powers of two (|q'|^2 + |r'|^2 - 2 q'.r', TMEM accumulator) FILTERS the
 * references with a rigorous error bound eps_q (R21), keeping every
 * reference whose filter distance is within 2 eps_q of a k-th value, starting
 * from a speculative per-query bound (a sampled pre-pass of the same kernel,
 * verified afterwards); the survivors are rescored exactly and selected.  Queries
 * whose band of near-equal filter distances overflows a pool, whose speculative
 * bound fails its verification, or with non-finite inputs are solved by an exact
 * brute-force fallback on the device.
 * The Q x N distance matrix is never written to memory. */
KSEL_API size_t knn_search_workspace(int64_t N, int64_t Q, int D, int k);
KSEL_API int knn_search(const float* ref, const float* query, int64_t N, int64_t Q, int D, int k,
               float* out_dist, int32_t* out_idx, int64_t idx_offset, void* d_work,
               size_t work_bytes, void* stream);

/* knn_graph -- the k-nearest-neighbour graph of one point set (k-NNG
 * construction, the workload of QMS [9]): for
 * every point i of points[N][D], its k nearest OTHER points, i.e. the k
 * lexicographically smallest (d(i, j), j) over j != i, ascending.  Computed as
 * knn_search(points, points, k + 1) followed by removing i from row i (when i is
 * not among the k + 1 -- more than k duplicates of i with lower indices -- the
 * first k are the answer), so distances, ties and accuracy are those of
 * knn_search.
 *   points   device, N x D fp32 row-major (read only)
 *   out_dist device, N x k fp32 (squared L2); out_idx device, N x k int32
 *   d_work   device workspace of >= knn_graph_workspace(N, D, k) bytes
 * Errors: KSEL_ERR_INVALID_ARG for N < 2, k < 1, k > N - 1, null pointers or a
 * short workspace; KSEL_ERR_UNSUPPORTED for k + 1 > 1024 or D > 256. */
KSEL_API size_t knn_graph_workspace(int64_t N, int D, int k);
KSEL_API int knn_graph(const float* points, int64_t N, int D, int k, float* out_dist, int32_t* out_idx,
                       void* d_work, size_t work_bytes, void* stream);

/* knn_distances -- DIAGNOSTIC (not the hot path): the filter distances d~(q, r) of
 * knn_search's tensor-core pass (fp16 operands, fp32 accumulation, clamped at 0)
 * written to out[Q][N] (device, fp32) instead of being filtered, and, if out_eps
 * (device, [Q]) is not NULL, the bound eps_q with |d~(q, r) - d(q, r)| <= eps_q
 * for every r that knn_search relies on.  Lets tests pin the tensor-core
 * distance and its error bound against the oracle's definition.
 * Workspace from knn_distances_workspace(N, Q, D). */
KSEL_API size_t knn_distances_workspace(int64_t N, int64_t Q, int D);
KSEL_API int knn_distances(const float* ref, const float* query, int64_t N, int64_t Q, int D, float* out,
                           float* out_eps, void* d_work, size_t work_bytes, void* stream);

/* ksel_select_paper -- ABLATION, not the hot path: the
 * paper's own per-thread designs, one thread per query, on B200.
 *   dist_t   device, [N][Q] fp32: QUERY-CONTIGUOUS (element (q, j) at j*Q + q),
 *            the layout that makes a thread-per-query scan coalesced (PAPER.md
 *            L225, L243; reading R10).
 *   queue    KSEL_PQ_INSERT (sorted array, L37), KSEL_PQ_HEAP (L37),
 *            KSEL_PQ_MERGE (Merge Queue, Alg. 2, L39-L41, level-1 size m),
 *            KSEL_PQ_MERGE_ALIGNED (merges taken by the whole warp, L183).
 *   buffer   KSEL_PB_NONE, KSEL_PB_BUFFER / KSEL_PB_FULL / KSEL_PB_FULL_SORTED
 *            (Buffered Search, Alg. 3; bsize pairs per thread).
 *   hp_G     0, or the Hierarchical Partition group size G >= 2 (Alg. 4).
 *   d_work   device workspace >= ksel_select_paper_workspace(...) bytes (queues,
 *            buffers and HP levels per thread; 0 returned for invalid arguments).
 * Output as ksel_select (out_val/out_idx [Q][k], ascending, bit-identical for
 * every variant).  Errors: INVALID_ARG (bad variant, m not a power of 2 in
 * [1, 1024], bsize outside [1, 1024], G outside {0} U [2, 64], short workspace),
 * UNSUPPORTED (k > 1024). */
#define KSEL_PQ_INSERT 0
#define KSEL_PQ_HEAP 1
#define KSEL_PQ_MERGE 2
#define KSEL_PQ_MERGE_ALIGNED 3
#define KSEL_PB_NONE 0
#define KSEL_PB_BUFFER 1
#define KSEL_PB_FULL 2
#define KSEL_PB_FULL_SORTED 3
KSEL_API size_t ksel_select_paper_workspace(int64_t Q, int64_t N, int k, int queue, int buffer, int hp_G, int m,
                                            int bsize);
KSEL_API int ksel_select_paper(const float* dist_t, int64_t Q, int64_t N, int k, int queue, int buffer, int hp_G,
                               int m, int bsize, float* out_val, int32_t* out_idx, void* d_work, size_t work_bytes,
                               void* stream);

/* ---- Row-sharded k-NN exchange without a collective ----
 * The final merge of the row-sharded k-NN (divide-and-merge)
 * reading every shard's candidate lists in place -- local memory or a peer
 * GPU's memory mapped over NVLink with CUDA IPC -- with stream-ordered
 * device-side release/acquire flags instead of an NCCL all-gather + host
 * barrier.  Orchestration (double buffering, epochs): dist.py KnnP2P.
 *
 * ksel_ipc_alloc -- cudaMalloc `bytes` (zero-filled) and export it: *d_ptr is the
 *   device pointer, handle_out receives ksel_ipc_handle_size() bytes (a
 *   cudaIpcMemHandle_t) that another process maps with ksel_ipc_open.  The
 *   caller owns the allocation (ksel_ipc_free).  KSEL_ERR_CUDA on failure.
 * ksel_ipc_open / ksel_ipc_close -- map / unmap another process's allocation
 *   (cudaIpcOpenMemHandle with lazy peer access; not for the exporting process
 *   itself, which uses its own pointer).
 * ksel_flag_signal -- enqueue on `stream`: after all earlier work of the stream,
 *   a system-scope fence then a release store of `value` to the u32 *d_flag
 *   (local or peer memory, 4-byte aligned).
 * ksel_flag_wait -- enqueue on `stream`: later work of the stream starts only
 *   after every d_flags[j] (j < n <= 64, device pointers, local or peer) holds
 *   a value v with (int32)(v - value) >= 0 (acquire at system scope).  The
 *   pointer array itself is host memory, read during the call.
 * ksel_merge_lists -- ksel_merge over S <= 64 lists given as pointer tables
 *   (host arrays of device pointers): list s of query q (0 <= q < Q) is
 *   vals[s] + q*kin / idxs[s] + q*kin, sorted ascending in (value, index) as
 *   knn_search emits it; indices unique per query across lists.  With ready
 *   != NULL, list s is read only after *ready[s] reached `epoch` (as in
 *   ksel_flag_wait), with volatile loads.  Output, limits and errors as
 *   ksel_merge.
 * A wait that does not complete within the flag timeout (ksel_set_flag_timeout,
 * default 600 s) gives up instead of hanging: the waiting kernel records
 * KSEL_ERR_TIMEOUT in a library-owned word of mapped host memory and returns
 * (the CUDA context stays usable; the results of that exchange are invalid).
 * ksel_device_status() -- call it after synchronising the stream -- returns
 * KSEL_OK or KSEL_ERR_TIMEOUT; ksel_device_status_clear() resets it.  Every
 * kernel taking part in such an exchange must already be loaded when a wait is
 * pending (CUDA lazy loading may otherwise serialise behind the spinning wait):
 * run one warm-up call first, as KnnP2P does. */
KSEL_API size_t ksel_ipc_handle_size(void);
KSEL_API int ksel_ipc_alloc(size_t bytes, void** d_ptr, void* handle_out);
KSEL_API int ksel_ipc_open(const void* handle, void** d_ptr);
KSEL_API int ksel_ipc_close(void* d_ptr);
KSEL_API int ksel_ipc_free(void* d_ptr);
KSEL_API int ksel_flag_signal(uint32_t* d_flag, uint32_t value, void* stream);
KSEL_API int ksel_flag_wait(const uint32_t* const* d_flags, int n, uint32_t value, void* stream);
KSEL_API int ksel_merge_lists(const float* const* vals, const int32_t* const* idxs, int S, int64_t Q, int kin,
                              int k, float* out_val, int32_t* out_idx, const uint32_t* const* ready,
                              uint32_t epoch, void* stream);
/* seconds > 0: flag-wait timeout of waits enqueued from now on (KSEL_ERR_INVALID_ARG otherwise). */
KSEL_API int ksel_set_flag_timeout(double seconds);
KSEL_API int ksel_device_status(void);
KSEL_API int ksel_device_status_clear(void);

/* Live per-kernel timing (measurement support for bench.py): while enabled,
 * every entry point records a pair of CUDA events on its stream around its
 * DOMINANT kernel (ksel_select: the selection kernel; knn_search: the fused
 * distance+selection kernel).  ksel_timing_collect synchronises those events,
 * returns the summed milliseconds and the number of launches timed, and
 * clears the record.  Off by default (no events, no overhead). */
KSEL_API int ksel_timing_enable(int on);
KSEL_API int ksel_timing_collect(double* total_ms, int64_t* launches);

/* Human-readable text for a ksel_status (static storage, never NULL). */
KSEL_API const char* ksel_strerror(int status);

/* Library version, encoded as major*10000 + minor*100 + patch. */
KSEL_API int ksel_version(void);

/* Number of device kernels this library has enqueued since load (all entry
 * points, all threads).  Used by bench.py to report gpu_launches. */
KSEL_API int64_t ksel_launch_count(void);

#ifdef __cplusplus
}
#endif

#endif /* KSEL_H_ */
