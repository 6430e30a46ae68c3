// knn_common.cuh -- shared definitions of the fused k-NN filter (knn_fused.cu) and its
// exact rescoring / fallback kernels (knn_rescore.cu).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ksel {

constexpr int KNN_MAX_D = 256;

// Maxima over the reference set (non-negative floats as bits; reset per call).
struct KnnStats {
    uint32_t R2;    // max |r'|^2 of the centred references (rounded up)
    uint32_t isig;  // max 1 / sigma_t over the reference tiles
    uint32_t pad[2];
};

// eps_q: a rigorous bound on |d~(q, r) - d(q, r)| for every reference r, where d~ is the
// filter's tensor-core distance and d the exact one (reading R21).  The filter
// (knn_fused.cu) centres every point (x' = fl(x - c)), scales each tile by a power of two
// sigma and rounds to fp16: A = fp16(-2 sigma_q q'), B = fp16(sigma_t r'), one kind::f16
// MMA pass; the norms |q'|^2, |r'|^2 (double, rounded to fp32, split three ways in bf16)
// ride in the same fp32 accumulation.  qs = (sigma_q, -, -, |q'|^2), na = |q'|^2, R2 = max
// |r'|^2.  In unscaled units:
//   * operand rounding: each fp16 operand is off by <= 2^-11 of itself (normal) or 2^-25
//     absolute (subnormal); a product -2 q'_i r'_i is off by <= (2^-10 + 2^-22) |2 q'_i r'_i|
//     plus 2^-25 (|A_i| + |B_i|) / (sigma_q sigma_t) <= 2^-9 / (sigma_q sigma_t) (|A|, |B|
//     <= 2^15), and sum |q'_i r'_i| <= |q'| |r'| <= sqrt(na R2):
//     2 (2^-10 + 2^-21) sqrt(na R2) + D 2^-9 / (sigma_q sigma_t,min);
//   * fp32 accumulation of D products and 6 norm terms, each rounding <= 2^-24 of the
//     absolute sum <= 2.02 (na + |r'|^2): (D + 16) 2^-23 1.01 (na + R2), plus
//     (D + 16) 2^-124 / (sigma_q sigma_t,min) for underflow;
//   * centring (|fl(x - c) - (x - c)| <= 2^-24 |x'|, so d' = |q' - r'|^2 is within
//     2^-22 (na + |r'|^2) of d) and the 24-bit norm splits: 2^-21 (na + R2);
// times 2 for safety.  Returned rounded up; +Inf if an input is not finite (the query
// then takes the exact fallback).
__device__ __forceinline__ float knn_eps(float4 qs, const KnnStats& st, int D) {
    const double R2 = (double)__uint_as_float(st.R2), nq = (double)qs.w;
    const double isq = (double)__uint_as_float(st.isig) / (double)qs.x;  // 1 / (sigma_q sigma_t,min)
    const double e = 2.0 * ((0x1p-10 + 0x1p-21) * 2.0 * sqrt(nq * R2) + (double)(D + 16) * 0x1p-23 * 1.01 * (nq + R2) +
                            0x1p-21 * (nq + R2) + ((double)D * 0x1p-9 + (double)(D + 16) * 0x1p-124) * isq);
    const float f = __double2float_ru(e);
    return (f == f) ? f : __int_as_float(0x7f800000);
}

// Exact brute-force fallback (queries whose band overflowed a pool): kFbCtas CTAs of
// kFbWarps warps; per CTA a global-memory pool of k' + 256 exact pairs per warp and a
// merge area of kFbWarps * k' pairs.
constexpr int kFbCtas = 64;
constexpr int kFbWarps = 8;
__host__ __device__ constexpr int knn_queue(int k) {
    return k <= 32 ? 32 : k <= 64 ? 64 : k <= 128 ? 128 : k <= 256 ? 256 : k <= 512 ? 512 : 1024;
}
__host__ __device__ constexpr size_t knn_fallback_bytes(int k) {
    return (size_t)kFbCtas * (size_t)kFbWarps * (size_t)(2 * knn_queue(k) + 256) * 8u;
}

struct KnnRescoreArgs {
    const float* ref;
    const float* query;   // this chunk's queries
    int64_t N, Q;
    int D, k;
    int64_t idx_offset;
    const unsigned long long* pools;  // [S][Q][P] packed (key(d~) << 32 | ref row)
    int64_t P;
    const int32_t* cnt;                // [S][Q]
    int S;                             // lists per query (reference splits x column halves)
    const unsigned long long* thr;     // [Q] tightest published k-th (d~, row) pair
    int32_t* qfail;                    // [Q] band overflowed / speculation unverified: exact fallback
    const unsigned long long* spec;    // [Q] speculative starting bound T_spec (nullptr: none)
    const float4* qstat;               // [Q] (-, -, -, |q|^2)
    const KnnStats* stats;
    uint8_t* fb;                       // fallback workspace
    float* out_val;
    int32_t* out_idx;
    unsigned long long* cand;          // [Q][kCandCap] the band of each query (rescore -> exact -> finish)
    int32_t* ccount;                   // [Q] its length; -1: finished (phase B) or flagged
};
constexpr int kCandCap = 1600;         // the largest rescore buffer (k' = 1024: k + the band)

// knn_rescore.cu
cudaError_t launch_knn_rescore(const KnnRescoreArgs& a, cudaStream_t stream);
cudaError_t launch_knn_fallback(const KnnRescoreArgs& a, cudaStream_t stream);
template <int R>
cudaError_t launch_knn_rescore_r(const KnnRescoreArgs& a, cudaStream_t stream);
template <int R>
cudaError_t launch_knn_fallback_r(const KnnRescoreArgs& a, cudaStream_t stream);

}  // namespace ksel
