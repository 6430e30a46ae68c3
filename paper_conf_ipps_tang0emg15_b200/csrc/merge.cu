// KSEL_SPLIT_R
// merge.cu -- ksel_merge: per-query merge of S sorted candidate lists.
//
// The final step of divide-and-merge (ref. [18]) and of the
// row-sharded k-NN after the NCCL all-gather.  One warp per
// query keeps a register-resident sorted queue of k' = max(32, 2^ceil(log2 k))
// pairs; each list is merged in with the Reverse Bitonic Merge "flip" + clean
// (Fig. 2; Merge Queue levels merged lazily, L41).  Lists are
// checked for sortedness with one neighbour compare per element and sorted in
// the warp if a caller hands in an unsorted list, so the result is the exact
// top-k of the union either way.
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel_common.cuh"
#include "ksel_internal.h"
#include "ksel_pool.cuh"

#ifndef KSEL_ONLY_R
#error "compile once per queue size with -DKSEL_ONLY_R=1|2|4|8|16|32"
#endif

namespace ksel {

constexpr int kMergeWarps = 4;

template <int RL>
__device__ __forceinline__ bool warr_is_sorted(const WArr<RL>& a, uint32_t lane) {
    bool bad = false;
#pragma unroll
    for (int r = 0; r < RL; ++r) {
        uint32_t nk = __shfl_down_sync(kFull, a.k[r], 1);
        uint32_t ni = __shfl_down_sync(kFull, a.i[r], 1);
        if (r + 1 < RL) {
            const uint32_t hk = __shfl_sync(kFull, a.k[r + 1], 0);
            const uint32_t hi = __shfl_sync(kFull, a.i[r + 1], 0);
            if (lane == 31) { nk = hk; ni = hi; }
        }
        const bool has_next = (lane < 31) || (r + 1 < RL);
        bad |= has_next && pair_lt(nk, ni, a.k[r], a.i[r]);
    }
    return !__any_sync(kFull, bad);
}

// Loads of list elements: through the read-only path for local lists; for lists in
// a peer's memory that are re-filled every step (ksel_merge_lists with ready flags),
// volatile (.cv) loads, so no stale line of an earlier step is ever used.
__device__ __forceinline__ float ld_val(const MergeLists& L, const float* p) { return L.vol ? __ldcv(p) : __ldg(p); }
__device__ __forceinline__ int32_t ld_idx(const MergeLists& L, const int32_t* p) { return L.vol ? __ldcv(p) : __ldg(p); }

// Wait (one lane, acquire at system scope) until list s of this step is published.
__device__ __forceinline__ void wait_ready(const MergeLists& L, int s) {
    if (L.ready[s] == nullptr) return;
    if (lane_id() == 0) {
        uint32_t v;
        const uint64_t t0 = globaltimer_ns();
        while (true) {
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(L.ready[s]) : "memory");
            if ((int32_t)(v - L.epoch) >= 0) break;
            __nanosleep(256);
            if (globaltimer_ns() - t0 > L.timeout_ns) {  // a producer that never signals: give up, report
                note_timeout(L.err);
                break;
            }
        }
    }
    __syncwarp();
}

// Bits of the candidate (key, idx) of query q in the S lists: lanes take
// lists, binary search for the lexicographic lower bound of (key, idx) in a sorted
// list (8-10 dependent loads); a warp-wide linear scan if no list has it at the
// searched position (unsorted input lists).  Warp-uniform result.
static __device__ __noinline__ uint32_t regather_bits(const MergeLists& L, int64_t q, int S, int kin, uint32_t key,
                                                      uint32_t idx, uint32_t lane) {
    for (int s0 = 0; s0 < S; s0 += 32) {
        const int s = s0 + (int)lane;
        bool hit = false;
        uint32_t hb = 0;
        if (s < S) {
            const float* cv = L.v[s] + q * kin;
            const int32_t* ci = L.i[s] + q * kin;
            int lo = 0, hi = kin;  // first position not below (key, idx)
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (pair_lt(key_of(ld_val(L, cv + mid)), (uint32_t)ld_idx(L, ci + mid), key, idx)) lo = mid + 1;
                else hi = mid;
            }
            if (lo < kin && (uint32_t)ld_idx(L, ci + lo) == idx && key_of(ld_val(L, cv + lo)) == key) {
                hit = true;
                hb = __float_as_uint(ld_val(L, cv + lo));
            }
        }
        const uint32_t m = __ballot_sync(kFull, hit);
        if (m) return __shfl_sync(kFull, hb, __ffs(m) - 1);
    }
    const int64_t total = (int64_t)S * kin;
    for (int64_t t0 = 0; t0 < total; t0 += 32) {
        const int64_t t = t0 + lane;
        bool hit = false;
        uint32_t hb = 0;
        if (t < total) {
            const int64_t a = q * kin + t % kin;
            const int s = (int)(t / kin);
            hit = (uint32_t)ld_idx(L, L.i[s] + a) == idx && key_of(ld_val(L, L.v[s] + a)) == key;
            hb = __float_as_uint(ld_val(L, L.v[s] + a));
        }
        const uint32_t m = __ballot_sync(kFull, hit);
        if (m) return __shfl_sync(kFull, hb, __ffs(m) - 1);
    }
    return bits_of_key(key);  // not reached: the pair came from the lists
}

template <int R, int RL>
__global__ void __launch_bounds__(32 * kMergeWarps)
    ksel_merge_kernel(const __grid_constant__ MergeLists L, int64_t Q, int S, int kin, int k,
                      float* __restrict__ out_val, int32_t* __restrict__ out_idx) {
    const uint32_t lane = lane_id();
    const int64_t q = (int64_t)blockIdx.x * kMergeWarps + (threadIdx.x >> 5);
    if (q >= Q) return;
    constexpr int LN = 32 * RL;  // list elements merged per step (<= k')

    WArr<R> acc;
    warr_fill_sentinel<R>(acc);
#pragma unroll 1
    for (int s = 0; s < S; ++s) {
        wait_ready(L, s);
        const float* cv = L.v[s] + q * kin;
        const int32_t* ci = L.i[s] + q * kin;
        // A list longer than k' is folded in whole, k' at a time (only its k'
        // smallest can matter, but finding them must not assume sortedness).
#pragma unroll 1
        for (int off = 0; off < kin; off += LN) {
            WArr<RL> b;
#pragma unroll
            for (int r = 0; r < RL; ++r) {
                const int e = off + r * 32 + (int)lane;
                b.k[r] = (e < kin) ? key_of(ld_val(L, cv + e)) : kSentKey;
                b.i[r] = (e < kin) ? (uint32_t)ld_idx(L, ci + e) : kSentIdx;
            }
            const bool sorted = (kin <= LN) && warr_is_sorted<RL>(b, lane);
            if (!sorted) warr_sort<RL>(b, lane);
            warr_merge<R, RL>(acc, b, lane);
        }
    }

    float* ov = out_val + q * (int64_t)k;
    int32_t* oi = out_idx + q * (int64_t)k;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + (int)lane;
        const uint32_t key = acc.k[r];
        const uint32_t idx = acc.i[r];
        uint32_t bits = bits_of_key(key);
        // -0.0 / NaN payloads: the canonical key dropped the bits; find the candidate's
        // own copy, warp-cooperatively, one such output at a time (rare)
        uint32_t need = __ballot_sync(kFull, e < k && key_needs_regather(key));
        while (need) {
            const int j = __ffs(need) - 1;
            need &= need - 1u;
            const uint32_t b = regather_bits(L, q, S, kin, __shfl_sync(kFull, key, j),
                                             __shfl_sync(kFull, idx, j), lane);
            if ((int)lane == j) bits = b;
        }
        if (e < k) {
            ov[e] = __uint_as_float(bits);
            oi[e] = (int32_t)idx;
        }
    }
}

template <int R, int RL>
static cudaError_t launch_merge_rl(const MergeLists& L, int64_t Q, int S, int kin, int k, float* ov, int32_t* oi,
                                   cudaStream_t stream) {
    const int64_t grid = (Q + kMergeWarps - 1) / kMergeWarps;
    ksel_merge_kernel<R, RL><<<(unsigned)grid, 32 * kMergeWarps, 0, stream>>>(L, Q, S, kin, k, ov, oi);
    note_launch();
    return cudaGetLastError();
}

template <int R>
cudaError_t launch_merge_r(const MergeLists& L, int64_t Q, int S, int kin, int k, float* ov, int32_t* oi,
                           cudaStream_t stream) {
    const int lp = kin <= 32 ? 1 : kin <= 64 ? 2 : kin <= 128 ? 4 : kin <= 256 ? 8 : kin <= 512 ? 16 : 32;
    const int rl = lp < R ? lp : R;
    switch (rl) {
        case 1: return launch_merge_rl<R, 1>(L, Q, S, kin, k, ov, oi, stream);
        case 2: if constexpr (R >= 2) return launch_merge_rl<R, 2>(L, Q, S, kin, k, ov, oi, stream); break;
        case 4: if constexpr (R >= 4) return launch_merge_rl<R, 4>(L, Q, S, kin, k, ov, oi, stream); break;
        case 8: if constexpr (R >= 8) return launch_merge_rl<R, 8>(L, Q, S, kin, k, ov, oi, stream); break;
        case 16: if constexpr (R >= 16) return launch_merge_rl<R, 16>(L, Q, S, kin, k, ov, oi, stream); break;
        case 32: if constexpr (R >= 32) return launch_merge_rl<R, 32>(L, Q, S, kin, k, ov, oi, stream); break;
    }
    return cudaErrorInvalidValue;
}

template cudaError_t launch_merge_r<KSEL_ONLY_R>(const MergeLists&, int64_t, int, int, int, float*, int32_t*,
                                                 cudaStream_t);

}  // namespace ksel
