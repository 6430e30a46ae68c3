// KSEL_SPLIT_R
// select_stream.cu -- streaming batched k-selection for sm_100a.
//
// One pass over each row of dist[Q][N] (Algorithm 1), with the
// paper's three ideas re-cast for a Blackwell warp:
//
//  a1 staging:   each warp streams its contiguous segment of the row through a
//                private S-stage shared-memory ring filled by 1-D TMA bulk
//                copies (cp.async.bulk ... mbarrier::complete_tx), one elected
//                lane issuing; coalescing requirement PAPER.md L15/L225.
//  a2 filter:    a candidate test against the running k-th pair -- first as a
//                plain fp32 compare (x <= tv, one FSETP per element), then, only
//                for warps holding a candidate, the exact lexicographic
//                (key, index) test; admitted pairs are compacted into a per-warp
//                buffer with __ballot_sync/__popc.  This is Buffered Search's
//                "Candidate Buffering" + "Intra-Warp Communication"
//                (Algorithm 3) with a warp vote instead of a
//                volatile shared flag.
//  a3 local sort:the full buffer is bitonic-sorted across the warp (Local Sort,
//                PAPER.md L187 Alg. 3 line 11).
//  a4 queue:     a register-resident, warp-distributed sorted queue of
//                k' = max(32, 2^ceil(log2 k)) pairs; the sorted buffer is merged
//                with the reverse-bitonic "flip" + clean (Merge Queue,
//                PAPER.md L39-L41, L139; "aligned merge" L183: every lane merges
//                together).  The new threshold is queue[k-1].
//  a6 row merge: with W warps per row, every warp filters with the tightest
//                threshold any warp of the row has published (shared-memory
//                atomicMin on the packed pair), and the W sorted queues are
//                merged pairwise in shared memory at the end (divide-and-merge,
//                PAPER.md L243).
//  a7 emit:      ascending (value, index); values are the input bits (keys are
//                inverted; canonicalised -0.0/NaN keys are re-gathered).
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel_common.cuh"
#include "ksel_internal.h"

#ifndef KSEL_ONLY_R
#error "compile once per queue size with -DKSEL_ONLY_R=1|2|4|8|16|32"
#endif

namespace ksel {

template <int R, int RB, int WPR, int RPC, int CH, int S>
struct StreamCfg {
    static constexpr int kQueue = 32 * R;      // k'
    static constexpr int kCap = 32 * RB;       // buffer capacity
    static constexpr int kWarps = WPR * RPC;
    static constexpr int kThreads = 32 * kWarps;
    static constexpr int kG = 2;               // float4 per lane per sub-step
    static constexpr int kRingBytes = S * CH * 4;
    // per warp: ring | queue keys, idx (k' each) | buffer keys, idx (cap each) | mbarriers
    static constexpr int kWarpBytes = kRingBytes + kQueue * 8 + kCap * 8 + S * 8;
    static constexpr int kWarpStride = (kWarpBytes + 127) / 128 * 128;
    static constexpr int kGroupBytes = 128;    // per row group: shared threshold
    static constexpr int kSmem = RPC * kGroupBytes + kWarps * kWarpStride;
    static_assert(CH % 128 == 0, "chunk must be a multiple of 128 floats");
    static_assert((CH / 128) % kG == 0, "chunk sub-steps");
};

__device__ __forceinline__ void group_bar(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Local Sort + Merge Queue insert of the buffered candidates (PAPER.md L187
// Alg. 3 l.11-12; L39-L41, L139).  The queue lives in shared memory between
// flushes so the streaming loop keeps its registers; this is the only place it
// is held in registers.  Returns the new k-th pair packed as (key << 32 | idx).
template <int R, int RB>
__device__ __noinline__ unsigned long long flush_into_queue(uint32_t* __restrict__ qk, uint32_t* __restrict__ qi,
                                                            const uint32_t* __restrict__ bk,
                                                            const uint32_t* __restrict__ bi, int n, int k) {
    const uint32_t lane = lane_id();
    __syncwarp();
    WArr<RB> b;
#pragma unroll
    for (int r = 0; r < RB; ++r) {
        const int e = r * 32 + (int)lane;
        b.k[r] = (e < n) ? bk[e] : kSentKey;
        b.i[r] = (e < n) ? bi[e] : kSentIdx;
    }
    WArr<R> q;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        q.k[r] = qk[r * 32 + lane];
        q.i[r] = qi[r * 32 + lane];
    }
    warr_sort<RB>(b, lane);
    warr_merge<R, RB>(q, b, lane);
#pragma unroll
    for (int r = 0; r < R; ++r) {
        qk[r * 32 + lane] = q.k[r];
        qi[r * 32 + lane] = q.i[r];
    }
    uint32_t kk, ki;
    warr_get<R>(q, k - 1, kk, ki);
    __syncwarp();
    return ((unsigned long long)kk << 32) | ki;
}

// Row merge step: queue (qk, qi) <- the k' smallest of itself and (pk, pi).
template <int R>
__device__ __noinline__ void merge_queues(uint32_t* __restrict__ qk, uint32_t* __restrict__ qi,
                                          const uint32_t* __restrict__ pk, const uint32_t* __restrict__ pi) {
    const uint32_t lane = lane_id();
    WArr<R> q, b;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        q.k[r] = qk[r * 32 + lane];
        q.i[r] = qi[r * 32 + lane];
        b.k[r] = pk[r * 32 + lane];
        b.i[r] = pi[r * 32 + lane];
    }
    warr_merge<R, R>(q, b, lane);
#pragma unroll
    for (int r = 0; r < R; ++r) {
        qk[r * 32 + lane] = q.k[r];
        qi[r * 32 + lane] = q.i[r];
    }
    __syncwarp();
}

template <int R, int RB, int WPR, int RPC, int CH, int S>
__global__ void __launch_bounds__(StreamCfg<R, RB, WPR, RPC, CH, S>::kThreads)
    ksel_stream_kernel(const float* __restrict__ dist, int64_t Q, int64_t N, int k,
                       float* __restrict__ out_val, int32_t* __restrict__ out_idx) {
    using Cfg = StreamCfg<R, RB, WPR, RPC, CH, S>;
    extern __shared__ __align__(128) uint8_t smem[];

    const uint32_t lane = lane_id();
    const int warp = threadIdx.x >> 5;
    const int grp = warp / WPR;
    const int wig = warp % WPR;
    const int64_t row = (int64_t)blockIdx.x * RPC + grp;
    if (row >= Q) return;  // whole row group leaves together (only group barriers below)

    unsigned long long* grp_thr = reinterpret_cast<unsigned long long*>(smem + grp * Cfg::kGroupBytes);
    uint8_t* wbase = smem + RPC * Cfg::kGroupBytes + warp * Cfg::kWarpStride;
    float* ring = reinterpret_cast<float*>(wbase);
    uint32_t* qk = reinterpret_cast<uint32_t*>(wbase + Cfg::kRingBytes);
    uint32_t* qi = qk + Cfg::kQueue;
    uint32_t* bufk = qi + Cfg::kQueue;
    uint32_t* bufi = bufk + Cfg::kCap;
    uint64_t* mbar = reinterpret_cast<uint64_t*>(bufi + Cfg::kCap);

    // ---- row geometry: unaligned head/tail + 16-byte aligned body -----------
    const uint64_t g0 = (uint64_t)row * (uint64_t)N;
    const uint64_t g1 = g0 + (uint64_t)N;
    const uint64_t mis = ((reinterpret_cast<uintptr_t>(dist) >> 2) + g0) & 3u;
    uint64_t a0 = g0 + ((4u - mis) & 3u);
    if (a0 > g1) a0 = g1;
    const uint64_t a1 = a0 + ((g1 - a0) & ~3ull);
    const uint64_t nch = (a1 - a0 + CH - 1) / CH;
    const uint64_t c_begin = nch * wig / WPR;
    const uint64_t c_end = nch * (wig + 1) / WPR;
    const int nmine = (int)(c_end - c_begin);

    auto chunk_len = [&](uint64_t c) -> uint32_t {  // floats, multiple of 4
        const uint64_t s0 = a0 + c * CH;
        const uint64_t s1 = (s0 + CH < a1) ? s0 + CH : a1;
        return (uint32_t)(s1 - s0);
    };
    auto issue = [&](int li) {  // lane 0 only
        const uint64_t c = c_begin + li;
        const int st = li % S;
        const uint32_t bytes = chunk_len(c) * 4u;
        mbar_arrive_expect_tx(&mbar[st], bytes);
        bulk_g2s(ring + st * CH, dist + a0 + c * CH, bytes, &mbar[st]);
    };

    if (lane == 0) {
        for (int s = 0; s < S; ++s) mbar_init(&mbar[s], 1);
        fence_mbar_init();
        for (int li = 0; li < S && li < nmine; ++li) issue(li);
    }
    if (WPR > 1 && wig == 0 && lane == 0) *grp_thr = 0xffffffffffffffffull;
    __syncwarp();
    if (WPR > 1) group_bar(1 + grp, 32 * WPR);

    // ---- selection state ------------------------------------------------------
#pragma unroll
    for (int r = 0; r < R; ++r) {
        qk[r * 32 + lane] = kSentKey;
        qi[r * 32 + lane] = kSentIdx;
    }
    uint32_t Tk = kSentKey, Ti = kSentIdx;  // filter threshold (k-th pair bound)
    float tv = 0.f;
    bool fast = false;  // Tk below +Inf: plain fp32 compare pre-filter is exact
    int n = 0;          // buffered candidates (warp-uniform)

    auto tighten = [&](uint32_t kk, uint32_t ki) {
        if (pair_lt(kk, ki, Tk, Ti)) { Tk = kk; Ti = ki; }
        fast = Tk < 0xff800000u;
        tv = __uint_as_float(bits_of_key(Tk));
    };

    auto flush = [&]() {
        const unsigned long long t = flush_into_queue<R, RB>(qk, qi, bufk, bufi, n, k);
        n = 0;
        const uint32_t kk = (uint32_t)(t >> 32), ki = (uint32_t)t;
        tighten(kk, ki);
        if (WPR > 1 && lane == 0 && kk != kSentKey) atomicMin(grp_thr, t);
    };

    // exact admission of one element per lane (valid lanes only)
    auto offer = [&](bool valid, float x, uint32_t col) {
        const uint32_t key = key_of(x);
        bool adm = valid && pair_lt(key, col, Tk, Ti);
        uint32_t bal = __ballot_sync(kFull, adm);
        if (bal == 0u) return;
        if (n + __popc(bal) > Cfg::kCap) {
            flush();
            adm = adm && pair_lt(key, col, Tk, Ti);
            bal = __ballot_sync(kFull, adm);
        }
        if (adm) {
            const int pos = n + __popc(bal & lanemask_lt());
            bufk[pos] = key;
            bufi[pos] = col;
        }
        n += __popc(bal);
        __syncwarp();
    };

    // ---- unaligned head and tail (< 4 elements each), warp 0 of the group ------
    if (wig == 0) {
        const uint32_t nh = (uint32_t)(a0 - g0), nt = (uint32_t)(g1 - a1);
        bool valid = false;
        uint64_t g = 0;
        if (lane < nh) { valid = true; g = g0 + lane; }
        else if (lane < nh + nt) { valid = true; g = a1 + (lane - nh); }
        const float x = valid ? dist[g] : 0.f;
        offer(valid, x, (uint32_t)(g - g0));
    }

    // ---- streaming body ---------------------------------------------------------
    for (int li = 0; li < nmine; ++li) {
        const int st = li % S;
        const uint64_t c = c_begin + li;
        const uint32_t len = chunk_len(c);
        const uint32_t col0 = (uint32_t)(a0 + c * CH - g0);
        if (WPR > 1) {
            const unsigned long long sh = *reinterpret_cast<volatile unsigned long long*>(grp_thr);
            tighten((uint32_t)(sh >> 32), (uint32_t)sh);
        }
        mbar_wait(&mbar[st], (uint32_t)(li / S) & 1u);
        const float4* src = reinterpret_cast<const float4*>(ring + st * CH);
#pragma unroll 1
        for (int g = 0; g < CH / 128; g += Cfg::kG) {
            float4 v[Cfg::kG];
            bool any = false;
#pragma unroll
            for (int u = 0; u < Cfg::kG; ++u) {
                const uint32_t e4 = (uint32_t)(g + u) * 32u + lane;  // float4 slot in chunk
                const bool ok = e4 * 4u < len;
                v[u] = ok ? src[e4] : make_float4(__int_as_float(0x7fc00000), __int_as_float(0x7fc00000),
                                                  __int_as_float(0x7fc00000), __int_as_float(0x7fc00000));
                if (fast) {
                    any |= (v[u].x <= tv) | (v[u].y <= tv) | (v[u].z <= tv) | (v[u].w <= tv);
                } else {
                    any |= ok;
                }
            }
            if (__any_sync(kFull, any)) {
                // exact pass over the sub-step, re-reading the staged values
                const float* srcf = ring + st * CH;
#pragma unroll 1
                for (int t = 0; t < Cfg::kG * 4; ++t) {
                    const uint32_t e = (uint32_t)(g + (t >> 2)) * 128u + lane * 4u + (uint32_t)(t & 3);
                    const bool ok = e < len;
                    offer(ok, ok ? srcf[e] : 0.f, col0 + e);
                }
            }
        }
        __syncwarp();
        if (lane == 0 && li + S < nmine) issue(li + S);
    }
    if (n > 0) flush();

    // ---- merge the W warp queues of the row (pairwise, through shared memory) --
    if (WPR > 1) {
#pragma unroll 1
        for (int step = 1; step < WPR; step <<= 1) {
            group_bar(1 + grp, 32 * WPR);
            if ((wig & (2 * step - 1)) == 0) {
                const uint32_t* pk = reinterpret_cast<const uint32_t*>(
                    smem + RPC * Cfg::kGroupBytes + (warp + step) * Cfg::kWarpStride + Cfg::kRingBytes);
                merge_queues<R>(qk, qi, pk, pk + Cfg::kQueue);
            }
        }
        if (wig != 0) return;
    }

    // ---- emit ascending (value bits, index) --------------------------------------
    float* ov = out_val + row * (int64_t)k;
    int32_t* oi = out_idx + row * (int64_t)k;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + (int)lane;
        if (e < k) {
            const uint32_t key = qk[e];
            const uint32_t col = qi[e];
            const uint32_t bits = key_needs_regather(key) ? __float_as_uint(dist[g0 + col]) : bits_of_key(key);
            ov[e] = __uint_as_float(bits);
            oi[e] = (int32_t)col;
        }
    }
}

// ---------------------------------------------------------------------------
// host-side dispatch
// ---------------------------------------------------------------------------
template <int R, int RB, int WPR, int RPC, int CH, int S>
static cudaError_t launch_cfg(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi,
                              cudaStream_t stream) {
    using Cfg = StreamCfg<R, RB, WPR, RPC, CH, S>;
    auto kern = ksel_stream_kernel<R, RB, WPR, RPC, CH, S>;
    cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), Cfg::kSmem);
    if (e != cudaSuccess) return e;
    const int64_t grid = (Q + RPC - 1) / RPC;
    kern<<<(unsigned)grid, Cfg::kThreads, Cfg::kSmem, stream>>>(dist, Q, N, k, ov, oi);
    note_launch();
    return cudaGetLastError();
}

template <int R, int RB, int WPR, int RPC, int CH, int S>
static cudaError_t launch_fit(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi,
                              cudaStream_t stream) {
    if constexpr (StreamCfg<R, RB, WPR, RPC, CH, S>::kSmem > kMaxSmemPerBlock) {
        if constexpr (RPC > 1) return launch_fit<R, RB, WPR, RPC / 2, CH, S>(dist, Q, N, k, ov, oi, stream);
        else return launch_fit<R, RB, WPR / 2, 1, CH, S>(dist, Q, N, k, ov, oi, stream);
    } else {
        return launch_cfg<R, RB, WPR, RPC, CH, S>(dist, Q, N, k, ov, oi, stream);
    }
}

template <int R>
cudaError_t launch_stream_r(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int wpr,
                            cudaStream_t stream) {
    constexpr int CH = 1024, S = 4, RB = 2;
    switch (wpr) {
        case 1: return launch_fit<R, RB, 1, 4, CH, S>(dist, Q, N, k, ov, oi, stream);
        case 2: return launch_fit<R, RB, 2, 2, CH, S>(dist, Q, N, k, ov, oi, stream);
        case 4: return launch_fit<R, RB, 4, 1, CH, S>(dist, Q, N, k, ov, oi, stream);
        default: return launch_fit<R, RB, 8, 1, CH, S>(dist, Q, N, k, ov, oi, stream);
    }
}

template cudaError_t launch_stream_r<KSEL_ONLY_R>(const float*, int64_t, int64_t, int, float*, int32_t*, int,
                                                  cudaStream_t);

}  // namespace ksel
