// knn_fused.cu -- knn_search: tcgen05/TMEM distance GEMM fused with k-selection.
// (placeholder entry points until the fused kernel lands)
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_internal.h"

extern "C" {

size_t knn_search_workspace(int64_t N, int64_t Q, int D, int k) {
    (void)N; (void)Q; (void)D; (void)k;
    return 0;
}

int knn_search(const float* ref, const float* query, int64_t N, int64_t Q, int D, int k, float* out_dist,
               int32_t* out_idx, int64_t idx_offset, void* d_work, size_t work_bytes, void* stream) {
    (void)ref; (void)query; (void)N; (void)Q; (void)D; (void)k; (void)out_dist; (void)out_idx;
    (void)idx_offset; (void)d_work; (void)work_bytes; (void)stream;
    return KSEL_ERR_UNSUPPORTED;
}

}  // extern "C"
