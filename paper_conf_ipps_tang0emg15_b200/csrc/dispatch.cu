// dispatch.cu -- runtime k -> queue-size (R = k'/32) dispatch for the kernel
// families that build.py compiles once per R (select_stream, select_pool, merge).
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_internal.h"
#include "knn_common.cuh"

namespace ksel {

static int queue_regs(int k) {
    return k <= 32 ? 1 : k <= 64 ? 2 : k <= 128 ? 4 : k <= 256 ? 8 : k <= 512 ? 16 : 32;
}

int stream_warps_per_row(int64_t Q, int64_t N, int num_sms) {
    // enough warps to cover every SM several times, but >= 8 chunks per warp
    const int64_t target = (int64_t)num_sms * 12;
    int wpr = 1;
    while (wpr < 8 && Q * wpr < target && N / (1024 * (wpr * 2)) >= 8) wpr *= 2;
    return wpr;
}

int pool_launch_shape(int64_t Q, int64_t N, int k, int num_sms, int forced_wpr) {
    // Warps per row: spread short/few rows over more warps, but keep >= 128 k'
    // elements per warp (each warp's pool has to find its own k-th) and >= 8 chunks.
    const int kp = k <= 32 ? 32 : (k <= 64 ? 64 : (k <= 128 ? 128 : (k <= 256 ? 256 : (k <= 512 ? 512 : 1024))));
    int wpr = forced_wpr;
    if (wpr == 0) {
        wpr = 1;
        const int64_t seg_min = (int64_t)128 * kp > 4096 ? (int64_t)128 * kp : 4096;
        while (wpr < 8 && Q * wpr < (int64_t)num_sms * 12 && N / (wpr * 2) >= seg_min) wpr *= 2;
    }
    // Deep (6-stage) ring when every warp can be resident at ~19 KB of shared
    // memory each: more bytes in flight per warp when few warps share an SM.
    const bool deep = Q * wpr <= (int64_t)num_sms * 11;
    return deep ? -wpr : wpr;
}

#define KSEL_DISPATCH_R(FN, R_, ...)                  \
    switch (R_) {                                     \
        case 1: return FN<1>(__VA_ARGS__);            \
        case 2: return FN<2>(__VA_ARGS__);            \
        case 4: return FN<4>(__VA_ARGS__);            \
        case 8: return FN<8>(__VA_ARGS__);            \
        case 16: return FN<16>(__VA_ARGS__);          \
        default: return FN<32>(__VA_ARGS__);          \
    }

cudaError_t launch_select_stream(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int wpr,
                                 cudaStream_t stream) {
    KSEL_DISPATCH_R(launch_stream_r, queue_regs(k), dist, Q, N, k, ov, oi, wpr, stream)
}

cudaError_t launch_select_pool(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int wpr,
                               cudaStream_t stream, SegMap seg) {
    KSEL_DISPATCH_R(launch_pool_r, queue_regs(k), dist, Q, N, k, ov, oi, wpr, seg, stream)
}

cudaError_t launch_merge(const MergeLists& L, int64_t Q, int S, int kin, int k, float* ov, int32_t* oi,
                         cudaStream_t stream) {
    KSEL_DISPATCH_R(launch_merge_r, queue_regs(k), L, Q, S, kin, k, ov, oi, stream)
}

#ifdef KSEL_EXPERIMENTS
bool hist_supported(int64_t N, int k) { return N <= ((int64_t)1 << 30) && k >= 1 && k <= KSEL_MAX_K; }

cudaError_t launch_select_hist(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int sms,
                               cudaStream_t stream) {
    KSEL_DISPATCH_R(launch_hist_r, queue_regs(k), dist, Q, N, k, ov, oi, sms, stream)
}
#else
// KSEL_ALGO_HIST (select_hist.cu) is built into the experiments library only: it lost to
// the pool kernel on C2 (profiles/r02_c2_hist_kernel_exp.txt).
bool hist_supported(int64_t, int) { return false; }
cudaError_t launch_select_hist(const float*, int64_t, int64_t, int, float*, int32_t*, int, cudaStream_t) {
    return cudaErrorNotSupported;
}
#endif

cudaError_t launch_knn_rescore(const KnnRescoreArgs& a, cudaStream_t stream) {
    KSEL_DISPATCH_R(launch_knn_rescore_r, queue_regs(a.k), a, stream)
}

cudaError_t launch_knn_fallback(const KnnRescoreArgs& a, cudaStream_t stream) {
    KSEL_DISPATCH_R(launch_knn_fallback_r, queue_regs(a.k), a, stream)
}


}  // namespace ksel
