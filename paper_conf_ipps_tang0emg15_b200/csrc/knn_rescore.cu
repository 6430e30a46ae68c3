// KSEL_SPLIT_R
// knn_rescore.cu -- the exact end of knn_search (knn_fused.cu): rescoring of the
// candidates the fp16 tensor-core filter left, and an exact brute-force fallback.
//
// Every candidate's distance is recomputed in the oracle's own arithmetic (reading
// R9, the CPU definition in DESIGN.md section 2): d = (float) sum_{t < D} (q_t - r_t)^2
// with each difference and square in double and the sum taken in index order, one
// rounding to fp32 at the end (the differences and squares of fp32 inputs are exact
// in double, so only the additions round -- in the same order as the oracle).  The
// top-k by (d, index) of the exact pairs is then the oracle's result bit for bit
// (PAPER.md L13 distance phase, L11/L19 selection, L637 sorted output).
//
// knn_rescore_kernel: one warp per query.  The filter kernel left, per reference
// split, a pool of (d~, row) pairs holding every row with d~ <= T + 2 eps_q (T: any
// k-th d~).  The warp gathers the pools' pairs into a shared-memory buffer, narrowing
// it to the band above ITS k-th d~ (the k-th over all splits: tighter than any one
// split's), rescores the band (one lane per candidate) and keeps the exact top-k; if
// the band itself does not fit the buffer (k near 1024 with a wide band), candidates
// are rescored as they are gathered against the running exact k-th instead.
//
// knn_fallback_kernel: queries flagged by the filter (a band of tied d~ larger than
// the pool, or non-finite inputs) are solved by brute force: one CTA per query, every
// reference rescored exactly, per-warp pools of exact pairs narrowed by radix select,
// merged, sorted.  Slow (a full exact pass over N) but exact; it does nothing when no
// query is flagged.
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel_common.cuh"
#include "ksel_internal.h"
#include "ksel_pool.cuh"
#include "knn_common.cuh"

#ifndef KSEL_ONLY_R
#error "compile once per queue size with -DKSEL_ONLY_R=1|2|4|8|16|32"
#endif

namespace ksel {

// warps (queries) per block: 3 for k' = 1024 (its 12.8 KB buffers), else 4
__host__ __device__ constexpr int rs_warps(int R) { return R >= 32 ? 3 : 4; }
// exact-pair buffer per warp: 32 x rs_regs(R) pairs (>= k' + 32 for the queue k' = 32 R),
// sized per queue so that small k keeps registers (the narrowing's) and occupancy up
__host__ __device__ constexpr int rs_regs(int R) { return R <= 4 ? 12 : R <= 8 ? 16 : R <= 16 ? 24 : 36; }
// buffer capacity: k' = 1024 needs room for k + the band (C5: ~1250 pairs) -- beyond the
// register narrowing's 32 x 36, narrowings there use the shared-histogram radix select
__host__ __device__ constexpr int rs_cap(int R) { return R >= 32 ? kCandCap : 32 * rs_regs(R); }

// the want-th pair of buf[0, n) (band >= 0: keep the band above it), in place
template <int NR, bool GLOBAL>
__device__ __forceinline__ unsigned long long narrow_any(unsigned long long* buf, int n, uint32_t want, int* nn,
                                                         uint32_t* hist, float band = -1.f) {
    if (n <= 32 * NR) return pool_narrow64<NR, GLOBAL>(buf, n, want, nn, band);
    return pool_select64<GLOBAL>(buf, n, want, hist, nn, band);
}

// The oracle's distance of one reference row (r: D floats, global) to the query held in
// double (qd, shared memory): differences and squares in double, summed in index order.
__device__ __forceinline__ float exact_dist(const float* __restrict__ r, const double* __restrict__ qd, int D) {
    double acc = 0.0;
    if ((D & 3) == 0 && (reinterpret_cast<uintptr_t>(r) & 15u) == 0) {
        // 8 independent 16-byte loads in flight before any use (the row is a gather from
        // HBM / L2; a load-use chain per float4 would serialise on memory latency)
        const float4* r4 = reinterpret_cast<const float4*>(r);
        for (int t4 = 0; t4 < D / 4; t4 += 8) {
            float4 v[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) v[j] = (t4 + j < D / 4) ? __ldg(r4 + t4 + j) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                if (t4 + j < D / 4) {
                    const int t = 4 * (t4 + j);
                    double d = __dsub_rn(qd[t], (double)v[j].x);
                    acc = __dadd_rn(acc, __dmul_rn(d, d));
                    d = __dsub_rn(qd[t + 1], (double)v[j].y);
                    acc = __dadd_rn(acc, __dmul_rn(d, d));
                    d = __dsub_rn(qd[t + 2], (double)v[j].z);
                    acc = __dadd_rn(acc, __dmul_rn(d, d));
                    d = __dsub_rn(qd[t + 3], (double)v[j].w);
                    acc = __dadd_rn(acc, __dmul_rn(d, d));
                }
            }
        }
    } else {
        for (int t = 0; t < D; ++t) {
            const double d = __dsub_rn(qd[t], (double)__ldg(r + t));
            acc = __dadd_rn(acc, __dmul_rn(d, d));
        }
    }
    return __double2float_rn(acc);
}

__device__ __forceinline__ float key_value(uint32_t key) { return __uint_as_float(bits_of_key(key)); }

template <int R>
__device__ __forceinline__ void emit_sorted(const unsigned long long* buf, int c, int k, int64_t idx_offset,
                                            float* __restrict__ ov, int32_t* __restrict__ oi, uint32_t lane) {
    WArr<R> a;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + (int)lane;
        const unsigned long long pr = (e < c) ? buf[e] : ~0ull;
        a.k[r] = (e < c) ? (uint32_t)(pr >> 32) : kSentKey;
        a.i[r] = (e < c) ? (uint32_t)pr : kSentIdx;
    }
    warr_sort<R>(a, lane);
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + (int)lane;
        if (e < k) {
            // exact distances are >= +0 or NaN: the key inverts exactly except NaN payloads
            ov[e] = __uint_as_float(a.k[r] == 0xffffffffu ? 0x7fc00000u : bits_of_key(a.k[r]));
            oi[e] = (a.i[r] == kSentIdx) ? (int32_t)kSentIdx : (int32_t)((int64_t)a.i[r] + idx_offset);
        }
    }
}

// A bound on the want-th smallest KEY (d~) over the union of a query's S pools (global
// memory): min / max (and, fused in, the count of pairs <= ts -- the speculative bound's
// verification), then 8-bit histograms of the keys below their common prefix (MSD radix
// select [12], the per-warp histogram in shared memory, hist_find: ksel_pool.cuh) until the
// bucket holding the want-th key has <= 64 keys; its upper edge is returned (>= want keys
// are <= it, at most that bucket's keys lie between).  Usually one histogram pass for
// k <= 128, two for k = 1024.  *le_out = #{pairs <= ts}.
static __device__ __noinline__ uint32_t lists_kth_key(const unsigned long long* __restrict__ pools, const int32_t* __restrict__ cnt,
                                              int S, int64_t Q, int64_t q, int64_t P, uint32_t want,
                                              uint32_t* __restrict__ hist, unsigned long long ts, int* le_out) {
    const uint32_t lane = lane_id();
    auto scan = [&](auto f) {
        for (int s = 0; s < S; ++s) {
            const int ns = cnt[(int64_t)s * Q + q];
            const unsigned long long* pr = pools + ((int64_t)s * Q + q) * P;
            for (int base = 0; base < ns; base += 256) {
                unsigned long long v[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const int x = base + j * 32 + (int)lane;
                    v[j] = (x < ns) ? __ldcg(pr + x) : ~0ull;
                }
#pragma unroll
                for (int j = 0; j < 8; ++j)
                    if (base + j * 32 + (int)lane < ns) f(v[j]);
            }
        }
    };
    uint32_t kmin = 0xffffffffu, kmax = 0u;
    int le = 0;
    scan([&](unsigned long long pr) {
        const uint32_t kk = (uint32_t)(pr >> 32);
        kmin = min(kmin, kk);
        kmax = max(kmax, kk);
        le += (pr <= ts) ? 1 : 0;
    });
    kmin = __reduce_min_sync(kFull, kmin);
    kmax = __reduce_max_sync(kFull, kmax);
    *le_out = __reduce_add_sync(kFull, le);
    if (want == 0u) return 0u;
    int hi = (kmin == kmax) ? -1 : 31 - __clz(kmin ^ kmax);
    if (hi < 0) return kmin;
    uint32_t prefix = kmin & ~((2u << hi) - 1u);
    for (;;) {
        const int lo = hi >= 7 ? hi - 7 : 0;
        const uint32_t dmask = (2u << (hi - lo)) - 1u;
#pragma unroll
        for (int j = 0; j < 8; ++j) hist[j * 32 + lane] = 0u;
        __syncwarp();
        scan([&](unsigned long long pr) {
            const uint32_t kk = (uint32_t)(pr >> 32);
            if (hi == 31 || ((kk ^ prefix) >> (hi + 1)) == 0u) atomicAdd(&hist[hist_slot((kk >> lo) & dmask)], 1u);
        });
        __syncwarp();
        uint32_t cnt_b;
        const uint32_t d = hist_find(hist, lane, want, cnt_b);
        __syncwarp();
        prefix |= d << lo;
        // stop once the want-th key's bucket is small: its upper edge is then a bound with
        // few keys between it and the want-th (<= 64 extra candidates for the band)
        if (cnt_b <= 64u || lo == 0) return prefix | ((1u << lo) - 1u);
        hi = lo - 1;
    }
}

template <int R>
__global__ void __launch_bounds__(32 * rs_warps(R), 4) knn_rescore_kernel(const KnnRescoreArgs a) {
    constexpr int kRsWarps = rs_warps(R);
    constexpr int kRsRegs = rs_regs(R);
    constexpr int kRsCap = rs_cap(R);
    __shared__ unsigned long long buf_all[kRsWarps][kRsCap];
    __shared__ double qd_all[kRsWarps][KNN_MAX_D];
    __shared__ uint32_t hist_all[kRsWarps][256];
    const uint32_t lane = lane_id();
    const int w = threadIdx.x >> 5;
    const int64_t q = (int64_t)blockIdx.x * kRsWarps + w;
    if (q >= a.Q) return;
    if (a.qfail[q]) {
        if (lane == 0) a.ccount[q] = -1;
        return;
    }
    unsigned long long* buf = buf_all[w];
    double* qd = qd_all[w];
    for (int t = (int)lane; t < a.D; t += 32) qd[t] = (double)a.query[q * a.D + t];
    __syncwarp();
    const float eps = knn_eps(a.qstat[q], *a.stats, a.D);
    const float band = __fmul_ru(2.f, eps);
    // the k-th d~ over ALL of the query's pools (at least k references have a d~ <= it):
    // only the band above it can hold the exact top-k
    unsigned long long T0 = a.thr[q];
    // (with a speculative start: gather against min(T_spec, thr) + band in ONE pass, count the
    // verification inline, and let the buffer's narrowing find the k-th -- no union scans)
    const unsigned long long ts = a.spec ? a.spec[q] : ~0ull;
    const bool spec = (uint32_t)(ts >> 32) != kSentKey;
    {
        int tot = 0;
        for (int s = (int)lane; s < a.S; s += 32) tot += a.cnt[(int64_t)s * a.Q + q];
        tot = __reduce_add_sync(kFull, tot);
        // A speculative start T_spec (knn_fused.cu knn_spec_geometry) made every split admit
        // against min(T_spec, its verified bounds).  The pools then hold every reference with
        // d~ <= min(T_spec, thr) + band, so the band may start from T_spec only once T_spec is
        // VERIFIED -- at least k pooled pairs <= T_spec -- or from thr if thr <= T_spec.
        // Otherwise the pools may miss part of the top-k: exact fallback.  (The count is taken
        // during the gather below; without a speculative bound a union larger than the buffer
        // is first bounded by a radix scan.)
        if (spec) {
            T0 = ts < T0 ? ts : T0;  // (provisional: verified after the gather)
        } else if (tot > kRsCap && tot >= a.k) {
            int le = 0;
            const uint32_t kk = lists_kth_key(a.pools, a.cnt, a.S, a.Q, q, a.P, (uint32_t)a.k, hist_all[w], ts, &le);
            {
                const unsigned long long t = ((unsigned long long)kk << 32) | 0xffffffffull;
                T0 = t < T0 ? t : T0;
            }
        }
    }
    unsigned long long Kb = band_bound(T0, band);  // candidates: pair <= Kb
    const uint32_t lt = lanemask_lt();
    // Phase A: gather the approximate pairs of all splits below the band, narrowing the
    // buffer to (its k-th d~ + the band) when it fills -- afterwards it holds exactly the
    // references that can be in the top-k.  Phase B (only if that band alone does not fit
    // the buffer): rescore what is there, keep the exact top-k, and from then on rescore
    // each gathered candidate at once, skipping those with d~ - eps_q above the exact k-th.
    bool exact_mode = false;
    unsigned long long Tx = ~0ull;            // exact bound (phase B)
    float txv = __int_as_float(0x7f800000);   // its value
    int c = 0;
    auto rescore_buffer = [&]() {
        for (int e = (int)lane; e < c; e += 32) {
            const uint32_t row = (uint32_t)buf[e];
            buf[e] = ((unsigned long long)key_of(exact_dist(a.ref + (int64_t)row * a.D, qd, a.D)) << 32) | row;
        }
        __syncwarp();
    };
    int le_spec = 0;  // pooled pairs <= T_spec (the speculative bound's verification)
    // one pair of the gather (phase A / B); x: its slot, ns: the list's length
    auto gather_one = [&](unsigned long long v, int x, int ns) {
            if (!exact_mode) {
                bool keep = x < ns && v <= Kb;
                uint32_t bal = __ballot_sync(kFull, keep);
                if (c + __popc(bal) > kRsCap) {
                    int nn;
                    const unsigned long long Ta = narrow_any<kRsRegs, false>(buf, c, (uint32_t)a.k, &nn, hist_all[w], band);
                    c = nn;
                    const unsigned long long Kn = band_bound(Ta, band);
                    Kb = Kn < Kb ? Kn : Kb;
                    keep = keep && v <= Kb;
                    bal = __ballot_sync(kFull, keep);
                    if (c + __popc(bal) > kRsCap) {  // the band alone overflows: phase B
                        rescore_buffer();
                        Tx = narrow_any<kRsRegs, false>(buf, c, (uint32_t)a.k, &nn, hist_all[w]);
                        c = nn;
                        txv = key_value((uint32_t)(Tx >> 32));
                        exact_mode = true;
                    }
                }
                if (!exact_mode) {
                    if (keep) buf[c + __popc(bal & lt)] = v;
                    c += __popc(bal);
                    __syncwarp();
                    return;
                }
            }
            // phase B: a candidate whose d~ - eps_q exceeds the exact k-th so far cannot win
            const bool cand = x < ns && v <= Kb && __fsub_rd(key_value((uint32_t)(v >> 32)), eps) <= txv;
            unsigned long long ex = ~0ull;
            if (cand) {
                const uint32_t row = (uint32_t)v;
                ex = ((unsigned long long)key_of(exact_dist(a.ref + (int64_t)row * a.D, qd, a.D)) << 32) | row;
            }
            bool keep = cand && ex <= Tx;
            uint32_t bal = __ballot_sync(kFull, keep);
            if (c + __popc(bal) > kRsCap) {  // full: narrow to the exact k-th pair
                int nn;
                Tx = narrow_any<kRsRegs, false>(buf, c, (uint32_t)a.k, &nn, hist_all[w]);
                c = nn;
                txv = key_value((uint32_t)(Tx >> 32));
                keep = keep && ex <= Tx;
                bal = __ballot_sync(kFull, keep);
            }
            if (keep) buf[c + __popc(bal & lt)] = ex;
            c += __popc(bal);
            __syncwarp();
    };
#pragma unroll 1
    for (int s = 0; s < a.S; ++s) {
        const int ns = a.cnt[(int64_t)s * a.Q + q];
        const unsigned long long* pr = a.pools + ((int64_t)s * a.Q + q) * a.P;
#pragma unroll 1
        for (int base = 0; base < ns; base += 128) {
            unsigned long long v[4];  // (4 loads in flight per lane)
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const int x = base + j * 32 + (int)lane;
                v[j] = (x < ns) ? __ldcg(pr + x) : ~0ull;
                le_spec += (x < ns && v[j] <= ts) ? 1 : 0;
            }
#pragma unroll 1
            for (int j = 0; j < 4 && base + j * 32 < ns; ++j) {
                const unsigned long long vj = j == 0 ? v[0] : j == 1 ? v[1] : j == 2 ? v[2] : v[3];  // (no local array)
                gather_one(vj, base + j * 32 + (int)lane, ns);
            }
        }
    }
    if (spec) {
        le_spec = __reduce_add_sync(kFull, le_spec);
        const unsigned long long thr = a.thr[q];
        if (le_spec < a.k && !(thr <= ts)) {  // T_spec not verified and no published bound below it
            if (lane == 0) { a.qfail[q] = 1; a.ccount[q] = -1; }
            return;
        }
    }
    if (!exact_mode) {  // phase A ended: the band set, rescored exactly by knn_exact_kernel
        if (c > a.k) {
            int nn;
            narrow_any<kRsRegs, false>(buf, c, (uint32_t)a.k, &nn, hist_all[w], band);
            c = nn;
        }
        unsigned long long* cq = a.cand + q * (int64_t)kCandCap;
        for (int e = (int)lane; e < c; e += 32) cq[e] = buf[e];
        if (lane == 0) a.ccount[q] = c;
        return;
    }
    if (lane == 0) a.ccount[q] = -1;  // (phase B finished this query here)
    if (c > a.k) {
        int nn;
        narrow_any<kRsRegs, false>(buf, c, (uint32_t)a.k, &nn, hist_all[w]);
        c = nn;
    }
    emit_sorted<R>(buf, c, a.k, a.idx_offset, a.out_val + q * a.k, a.out_idx + q * a.k, lane);
}

// knn_exact_kernel: the exact distances of every query's band (cand[q][0, ccount[q])), one
// warp per query, one lane per candidate row -- the register-light half of the rescoring
// (no narrowing / sorting state), so 32+ warps per SM keep the random 512-byte row
// gathers in flight (inside knn_rescore_kernel, at 16 warps per SM, they were latency-bound:
// C5 k = 1024, 2.9 ms).
template <int R>  // (R unused: one instantiation per compilation unit of this file)
__global__ void __launch_bounds__(256, 3) knn_exact_kernel(const KnnRescoreArgs a) {
    __shared__ double qd_all[8][KNN_MAX_D];
    const uint32_t lane = lane_id();
    const int w = threadIdx.x >> 5;
    const int64_t q = (int64_t)blockIdx.x * 8 + w;
    if (q >= a.Q) return;
    const int c = a.ccount[q];
    if (c <= 0) return;
    double* qd = qd_all[w];
    for (int t = (int)lane; t < a.D; t += 32) qd[t] = (double)a.query[q * a.D + t];
    __syncwarp();
    unsigned long long* cq = a.cand + q * (int64_t)kCandCap;
    for (int e = (int)lane; e < c; e += 32) {
        const uint32_t row = (uint32_t)cq[e];
        cq[e] = ((unsigned long long)key_of(exact_dist(a.ref + (int64_t)row * a.D, qd, a.D)) << 32) | row;
    }
}

// knn_finish_kernel: the exact top-k of each band (narrowing in global memory), sorted, emitted.
template <int R>
__global__ void __launch_bounds__(32 * rs_warps(R)) knn_finish_kernel(const KnnRescoreArgs a) {
    constexpr int kRsWarps = rs_warps(R);
    constexpr int kRsRegs = rs_regs(R);
    __shared__ uint32_t hist_all[kRsWarps][256];
    const uint32_t lane = lane_id();
    const int64_t q = (int64_t)blockIdx.x * kRsWarps + (threadIdx.x >> 5);
    if (q >= a.Q) return;
    int c = a.ccount[q];
    if (c < 0) return;
    unsigned long long* cq = a.cand + q * (int64_t)kCandCap;
    if (c > a.k) {
        int nn;
        narrow_any<kRsRegs, true>(cq, c, (uint32_t)a.k, &nn, hist_all[threadIdx.x >> 5]);
        c = nn;
        __syncwarp();
    }
    emit_sorted<R>(cq, c, a.k, a.idx_offset, a.out_val + q * a.k, a.out_idx + q * a.k, lane);
}

template <int R>
__global__ void __launch_bounds__(32 * kFbWarps) knn_fallback_kernel(const KnnRescoreArgs a) {
    __shared__ double qd[KNN_MAX_D];
    __shared__ uint32_t hist_all[kFbWarps][256];
    __shared__ int cnt_s[kFbWarps];
    constexpr int kp = 32 * R;
    constexpr int PW = kp + 256;  // per-warp pool
    const uint32_t lane = lane_id();
    const int w = threadIdx.x >> 5;
    const uint32_t lt = lanemask_lt();
    unsigned long long* cta = reinterpret_cast<unsigned long long*>(a.fb) +
                              (size_t)blockIdx.x * kFbWarps * (size_t)(2 * kp + 256);
    unsigned long long* wpool = cta + (size_t)w * PW;
    unsigned long long* merge = cta + (size_t)kFbWarps * PW;  // kFbWarps * kp pairs
    __shared__ int flagged[32 * kFbWarps];
    __shared__ int nflag;
    // scan the failure flags 256 at a time (one load per thread); solve the flagged queries
    for (int64_t q0 = (int64_t)blockIdx.x * 256; q0 < a.Q; q0 += (int64_t)gridDim.x * 256) {
        if (threadIdx.x == 0) nflag = 0;
        __syncthreads();
        const int64_t qq = q0 + threadIdx.x;
        if (qq < a.Q && a.qfail[qq]) flagged[atomicAdd(&nflag, 1)] = (int)threadIdx.x;
        __syncthreads();
        const int nf = nflag;
    for (int f = 0; f < nf; ++f) {
        const int64_t q = q0 + flagged[f];
        __syncthreads();
        for (int t = threadIdx.x; t < a.D; t += blockDim.x) qd[t] = (double)a.query[q * a.D + t];
        __syncthreads();
        unsigned long long Tw = ~0ull;
        int c = 0;
#pragma unroll 1
        for (int64_t i0 = (int64_t)w * 32; i0 < a.N; i0 += 32 * kFbWarps) {
            const int64_t i = i0 + lane;
            unsigned long long ex = ~0ull;
            if (i < a.N) ex = ((unsigned long long)key_of(exact_dist(a.ref + i * a.D, qd, a.D)) << 32) | (uint32_t)i;
            bool keep = i < a.N && ex <= Tw;
            uint32_t bal = __ballot_sync(kFull, keep);
            if (c + __popc(bal) > PW) {
                int nn;
                Tw = pool_select64(wpool, c, (uint32_t)a.k, hist_all[w], &nn);
                c = nn;
                keep = keep && ex <= Tw;
                bal = __ballot_sync(kFull, keep);
            }
            if (keep) wpool[c + __popc(bal & lt)] = ex;
            c += __popc(bal);
            __syncwarp();
        }
        if (c > a.k) {
            int nn;
            pool_select64(wpool, c, (uint32_t)a.k, hist_all[w], &nn);
            c = nn;
        }
        if (lane == 0) cnt_s[w] = c;
        __syncthreads();
        if (w == 0) {
            int m = 0;
            for (int v = 0; v < kFbWarps; ++v) {
                const int cv = cnt_s[v];
                const unsigned long long* src = cta + (size_t)v * PW;
                for (int e = (int)lane; e < cv; e += 32) merge[m + e] = __ldcg(src + e);
                m += cv;
            }
            __syncwarp();
            if (m > a.k) {
                int nn;
                pool_select64(merge, m, (uint32_t)a.k, hist_all[0], &nn);
                m = nn;
            }
            __syncwarp();
            // (merge is global memory: read it back through L2)
            WArr<R> s;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int e = r * 32 + (int)lane;
                const unsigned long long pr = (e < m) ? __ldcg(merge + e) : ~0ull;
                s.k[r] = (e < m) ? (uint32_t)(pr >> 32) : kSentKey;
                s.i[r] = (e < m) ? (uint32_t)pr : kSentIdx;
            }
            warr_sort<R>(s, lane);
            float* ov = a.out_val + q * a.k;
            int32_t* oi = a.out_idx + q * a.k;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int e = r * 32 + (int)lane;
                if (e < a.k) {
                    ov[e] = __uint_as_float(s.k[r] == 0xffffffffu ? 0x7fc00000u : bits_of_key(s.k[r]));
                    oi[e] = (int32_t)((int64_t)s.i[r] + a.idx_offset);
                }
            }
        }
        __syncthreads();
    }
    __syncthreads();
    }
}

template <int R>
cudaError_t launch_knn_rescore_r(const KnnRescoreArgs& a, cudaStream_t stream) {
    constexpr int kRsWarps = rs_warps(R);
    const int64_t grid = (a.Q + kRsWarps - 1) / kRsWarps;
    knn_rescore_kernel<R><<<(unsigned)grid, 32 * kRsWarps, 0, stream>>>(a);
    note_launch();
    knn_exact_kernel<R><<<(unsigned)((a.Q + 7) / 8), 256, 0, stream>>>(a);
    note_launch();
    knn_finish_kernel<R><<<(unsigned)grid, 32 * kRsWarps, 0, stream>>>(a);
    note_launch();
    return cudaGetLastError();
}

template <int R>
cudaError_t launch_knn_fallback_r(const KnnRescoreArgs& a, cudaStream_t stream) {
    const int64_t blocks = (a.Q + 255) / 256;
    const int grid = (int)(blocks < kFbCtas ? blocks : kFbCtas);
    knn_fallback_kernel<R><<<grid, 32 * kFbWarps, 0, stream>>>(a);
    note_launch();
    return cudaGetLastError();
}

template cudaError_t launch_knn_rescore_r<KSEL_ONLY_R>(const KnnRescoreArgs&, cudaStream_t);
template cudaError_t launch_knn_fallback_r<KSEL_ONLY_R>(const KnnRescoreArgs&, cudaStream_t);

}  // namespace ksel
