// knn_common.cuh -- shared definitions of the fused k-NN filter (knn_fused.cu) and its
// exact rescoring / fallback kernels (knn_rescore.cu).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ksel {

constexpr int KNN_MAX_D = 256;

// Maxima over the reference set (non-negative floats as bits; reset per call).
struct KnnStats {
    uint32_t R2;  // max |r|^2 (rounded up)
    uint32_t pad[3];
};

// eps_q: a rigorous bound on |d~(q, r) - d(q, r)| for every reference r, where d~ is the
// filter's tensor-core distance (bf16 hi/lo split operands, three MMA passes, norms
// folded into the fp32 accumulator; knn_fused.cu) and d the exact one (DESIGN.md
// reading R21).  qs = (-, -, -, |q|^2).
//   * x = hi + lo + res with |res| <= 2^-16 |x|, and the dropped lo.lo term is
//     <= 2^-16 (1 + 2^-7) |q_i r_i|: each product of the MMA operands (-2 q_i, r_i) is
//     off by <= 6.1 2^-16 |q_i r_i|, and sum |q_i r_i| <= |q| |r| <= sqrt(|q|^2 R2);
//   * fp32 accumulation of 3D products and 6 norm terms, each rounding <= 2^-24 of the
//     absolute sum <= 2.02 (|q|^2 + |r|^2), and the 24-bit norm splits:
//     (3D + 16) 2^-23 (|q|^2 + R2), plus (3D + 16) 2^-124 for underflow;
// times 2 for safety.  Returned rounded up; +Inf if an input is not finite (the query
// then takes the exact fallback).
__device__ __forceinline__ float knn_eps(float4 qs, const KnnStats& st, int D) {
    const double R2 = (double)__uint_as_float(st.R2), nq = (double)qs.w;
    // (+ (3D + 16) 2^-124: products and partial sums that underflow the fp32 range -- flushed
    // or denormal in the tensor core -- each lose less than 2^-126)
    const double e = 2.0 * (6.1 * 0x1p-16 * sqrt(nq * R2) + (double)(3 * D + 16) * 0x1p-23 * (nq + R2) +
                            (double)(3 * D + 16) * 0x1p-124);
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
};

// knn_rescore.cu
cudaError_t launch_knn_rescore(const KnnRescoreArgs& a, cudaStream_t stream);
cudaError_t launch_knn_fallback(const KnnRescoreArgs& a, cudaStream_t stream);
template <int R>
cudaError_t launch_knn_rescore_r(const KnnRescoreArgs& a, cudaStream_t stream);
template <int R>
cudaError_t launch_knn_fallback_r(const KnnRescoreArgs& a, cudaStream_t stream);

}  // namespace ksel
