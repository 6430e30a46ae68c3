// ksel_internal.h -- host-side declarations shared by the translation units of
// libksel.so (not part of the public ABI; see include/ksel.h).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ksel {

constexpr int kMaxSmemPerBlock = 227 * 1024;  // sm_100 opt-in dynamic shared memory per CTA

// Integer value of an environment variable, or `dflt` when unset/empty.  Only the
// experiment knobs (KSEL_* variables) read the environment; the defaults
// are the product.
int env_int(const char* name, int dflt);

// Chunk visit order of the streaming kernels (experiments only; env KSEL_ORDER):
// 0 = address order, 1 = spread prologue + address order, 2 = strided permutation (default).
int chunk_order_mode();

// Cached properties of the current device (mutex-protected; cudaGetDeviceProperties
// is far too slow to call per launch).  Returns a ksel_status.
struct DevInfo {
    int dev = -1;
    int sms = 0;
    int major = 0;
    int minor = 0;
};
int current_device_info(DevInfo* out);

// Raise a kernel's dynamic shared memory limit once per (function, device).
cudaError_t ensure_smem_attr(const void* func, int bytes);

// Dominant-kernel timing (ksel_timing_enable): bracket a launch on `stream`.
// timing_begin returns an opaque slot (or -1 when timing is off).
int timing_begin(cudaStream_t stream);
void timing_end(int slot, cudaStream_t stream);

// Count one enqueued kernel (reported through ksel_launch_count()).
void note_launch();

// Streaming selection (select_stream.cu).
int stream_warps_per_row(int64_t Q, int64_t N, int num_sms);
// Pool-kernel launch shape: warps per row, negative = deep (6-stage) ring.
int pool_launch_shape(int64_t Q, int64_t N, int k, int num_sms, int forced_wpr);
cudaError_t launch_select_stream(const float* dist, int64_t Q, int64_t N, int k, float* out_val,
                                 int32_t* out_idx, int wpr, cudaStream_t stream);

// Split-row mapping of the pool kernel (seg_len == 0: one virtual row per row).
struct SegMap {
    int64_t nseg = 1;     // segments per row
    int64_t seg_len = 0;  // columns per segment (the last one may be shorter)
};

// Pool + radix-narrowing selection (select_pool.cu).  With seg.seg_len > 0, Q counts
// virtual rows (segments x real rows).
cudaError_t launch_select_pool(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx,
                               int wpr, cudaStream_t stream, SegMap seg = SegMap());

// Cluster radix selection for rows of <= 65536 values (select_radix.cu).
bool radix_supported(int64_t N, int k);
cudaError_t launch_select_radix(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx,
                                cudaStream_t stream);

// One-CTA-per-row histogram selection for rows of <= 2^17 values (select_hist.cu).
bool hist_supported(int64_t N, int k);
cudaError_t launch_select_hist(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx,
                               int sms, cudaStream_t stream);
template <int R>
cudaError_t launch_hist_r(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int sms,
                          cudaStream_t stream);

// Merge of S sorted candidate lists (merge.cu).  List s of query q is
// v[s] + q * kin / i[s] + q * kin (lists may live in different allocations, e.g.
// peers' memory); ready[s] (optional) is waited for (>= epoch, acquire at system
// scope) before list s is read, vol selects volatile loads (re-filled peer lists).
constexpr int kMaxLists = 64;
struct MergeLists {
    const float* v[kMaxLists];
    const int32_t* i[kMaxLists];
    const uint32_t* ready[kMaxLists];
    uint32_t epoch;
    int vol;
    uint32_t* err;        // device view of the timeout word (ready != NULL only)
    uint64_t timeout_ns;  // flag-wait timeout
};

// Device-side flag waits give up after flag_timeout_ns() and OR KSEL_ERR_TIMEOUT's bit
// into a word of mapped (host) memory; device_error_word() is its device pointer
// (lazily created once per process; nullptr if the mapping failed).
uint32_t* device_error_word();
uint64_t flag_timeout_ns();
cudaError_t launch_merge(const MergeLists& L, int64_t Q, int S, int kin, int k, float* out_val, int32_t* out_idx,
                         cudaStream_t stream);


// Per-queue-size entry points (explicitly instantiated, one object per R).
template <int R>
cudaError_t launch_stream_r(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int wpr,
                            cudaStream_t stream);
template <int R>
cudaError_t launch_pool_r(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int wpr,
                          SegMap seg, cudaStream_t stream);
template <int R>
cudaError_t launch_merge_r(const MergeLists& L, int64_t Q, int S, int kin, int k, float* ov, int32_t* oi,
                           cudaStream_t stream);

}  // namespace ksel
