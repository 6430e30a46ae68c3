// KSEL_SPLIT_R
// select_pool.cu -- streaming k-selection with radix threshold narrowing (sm_100a).
//
// Same staging and filter as select_stream.cu (a1/a2: TMA bulk copies into a
// per-warp shared-memory ring, fp32 pre-filter against the running k-th pair,
// exact lexicographic test), but candidates are NOT merged into a sorted queue
// as they arrive.  They are appended, warp-aggregated, to an unordered
// per-warp candidate pool in shared memory (Buffered Search's candidate
// buffer, sized P >= k' + 256).  When the pool fills, an
// MSD radix-histogram select over the pool (8-bit digits of the order key,
// then of the index for ties) finds the exact k-th pair of everything seen so
// far; the pool is compacted to those k pairs and the pair becomes the new
// threshold.  This is the paper's Hierarchical Partition idea -- discard whole
// groups that cannot hold a k-NN ("if any element in the
// upper level does not belong to k-NN, none of the elements in its sub-groups
// would") -- with value buckets instead of index groups and a fixed number of
// steps (<= 8 digit passes) instead of log_G(N/k) (L231); radix select [12]
// (L15) is the digit order.
//
// At the end of the row the k surviving pairs are bitonic-sorted in the warp
// (Local Sort / Reverse Bitonic Merge networks), the
// W warps of a row are merged pairwise (divide-and-merge, L243), and the row's
// top-k is emitted ascending by (value, index).
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel_common.cuh"
#include "ksel_internal.h"
#include "ksel_pool.cuh"

#ifndef KSEL_ONLY_R
#error "compile once per queue size with -DKSEL_ONLY_R=1|2|4|8|16|32"
#endif

namespace ksel {

template <int R, int WPR, int RPC, int SD = 3>
struct PoolCfg {
    static constexpr int kQueue = 32 * R;  // k'
    // k' = 1024 with the shallow ring (many rows: shared memory limits the warps per SM):
    // k' + 512 pairs (one sub-step of room) -- 19 KB per warp instead of 23 KB, 11 warps
    // per SM instead of 9 (C3 k = 1024: 17.5 -> 15.7 ms).  With few rows (deep ring) the
    // larger pool's fewer narrowings win (C2 k = 1024: 0.24 vs 0.29 ms).
    static constexpr int kPool = (kQueue >= 1024 && SD <= 3)
                                     ? kQueue + 512
                                     : ((2 * kQueue > kQueue + 512) ? 2 * kQueue : kQueue + 512);
    static constexpr int CH = 512;         // floats per staged chunk (2 KB bulk copy)
    static constexpr int NB = (3 < SD) ? 3 : SD;  // chunks feeding the starting bound (1536 values)
    static constexpr int S = SD;           // ring stages per warp (3, or 6 when few warps run per SM)
    static constexpr int G = 4;            // float4 per lane per sub-step (512 elements per warp)
    static constexpr int NS = 4 * G;       // element slots per lane per sub-step
    static constexpr int kWarps = WPR * RPC;
    static constexpr int kThreads = 32 * kWarps;
    static constexpr int kRingBytes = S * CH * 4;
    // per warp: ring | pool keys | pool idx | histogram (256 u32) | mbarriers | stage chunk ids
    static constexpr int kWarpBytes = kRingBytes + kPool * 8 + 256 * 4 + S * 8 + S * 4;
    static constexpr int kWarpStride = (kWarpBytes + 127) / 128 * 128;
    static constexpr int kGroupBytes = 128;
    static constexpr int kSmem = RPC * kGroupBytes + kWarps * kWarpStride;
    static_assert(kPool % 32 == 0, "pool size");
    static_assert(kPool >= kQueue + 32 * NS, "a full sub-step must fit after compaction");
};

__device__ __forceinline__ void pool_group_bar(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// Sort pool[0..n) (n <= k') ascending into pool[0..k') with sentinel padding.
template <int R>
__device__ __noinline__ void pool_sort(uint32_t* __restrict__ pk, uint32_t* __restrict__ pi, int n) {
    const uint32_t lane = lane_id();
    WArr<R> a;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + (int)lane;
        a.k[r] = (e < n) ? pk[e] : kSentKey;
        a.i[r] = (e < n) ? pi[e] : kSentIdx;
    }
    __syncwarp();
    warr_sort<R>(a, lane);
#pragma unroll
    for (int r = 0; r < R; ++r) {
        pk[r * 32 + lane] = a.k[r];
        pi[r * 32 + lane] = a.i[r];
    }
    __syncwarp();
}

// Merge of two sorted k'-lists in shared memory: (qk, qi) <- k' smallest.
template <int R>
__device__ __noinline__ void pool_merge_sorted(uint32_t* __restrict__ qk, uint32_t* __restrict__ qi,
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

template <int R, int WPR, int RPC, int SD>
__global__ void __launch_bounds__(PoolCfg<R, WPR, RPC, SD>::kThreads, (R < 16 && WPR * RPC <= 16) ? 16 / (WPR * RPC) : 1)
    ksel_pool_kernel(const float* __restrict__ dist, int64_t Q, int64_t N, int k, float* __restrict__ out_val,
                     int32_t* __restrict__ out_idx, int order_mode, SegMap seg) {
    using Cfg = PoolCfg<R, WPR, RPC, SD>;
    constexpr int CH = Cfg::CH, S = Cfg::S, G = Cfg::G, NS = Cfg::NS;
    extern __shared__ __align__(128) uint8_t smem[];

    const uint32_t lane = lane_id();
    const int warp = threadIdx.x >> 5;
    const int grp = warp / WPR;
    const int wig = warp % WPR;
    const int64_t row = (int64_t)blockIdx.x * RPC + grp;
    if (row >= Q) return;

    unsigned long long* grp_thr = reinterpret_cast<unsigned long long*>(smem + grp * Cfg::kGroupBytes);
    uint8_t* wbase = smem + RPC * Cfg::kGroupBytes + warp * Cfg::kWarpStride;
    float* ring = reinterpret_cast<float*>(wbase);
    uint32_t* pk = reinterpret_cast<uint32_t*>(wbase + Cfg::kRingBytes);
    uint32_t* pi = pk + Cfg::kPool;
    uint32_t* hist = pi + Cfg::kPool;
    uint64_t* mbar = reinterpret_cast<uint64_t*>(hist + 256);
    uint32_t* cid = reinterpret_cast<uint32_t*>(mbar + S);  // chunk id of each stage

    // ---- row geometry -----------------------------------------------------------
    // Split rows (seg.seg_len > 0): virtual row v = q * seg.nseg + s is segment s
    // of row q, columns [s * seg_len, min(N, (s + 1) * seg_len)); its top-k goes to output
    // row v ([Q][S][k]: a row's S sorted lists are contiguous) with row-global indices.
    int64_t qrow = row;
    uint64_t coloff = 0, len = (uint64_t)N;
    if (seg.seg_len > 0) {
        qrow = row / seg.nseg;
        const int64_t sg = row - qrow * seg.nseg;
        coloff = (uint64_t)sg * (uint64_t)seg.seg_len;
        len = min((uint64_t)seg.seg_len, (uint64_t)N - coloff);
    }
    const uint64_t g0 = (uint64_t)qrow * (uint64_t)N + coloff;
    const uint64_t g1 = g0 + len;
    const uint64_t mis = ((reinterpret_cast<uintptr_t>(dist) >> 2) + g0) & 3u;
    uint64_t a0 = g0 + ((4u - mis) & 3u);
    if (a0 > g1) a0 = g1;
    const uint64_t a1 = a0 + ((g1 - a0) & ~3ull);
    const uint64_t nch = (a1 - a0 + CH - 1) / CH;
    const uint64_t c_begin = nch * wig / WPR;
    const uint64_t c_end = nch * (wig + 1) / WPR;
    const int nmine = (int)(c_end - c_begin);

    // Visit order of the warp's chunks (KSEL_ORDER; the result does not depend on it).
    // Default (3, r2): the first chunk, the last L = ceil(k / CH) + 1 chunks, then the
    // rest in column order.  The first and the last chunks feed the starting bound
    // (an ascending row's smallest values come first, a descending row's last; L covers
    // k of them), and the column-order remainder meets a tied row's smallest indices
    // first, so the exact (key, index) bound settles at once.  Measured against mode 2
    // (first, last, then a golden-ratio stride permutation, round 1's default): C2 tied
    // rows T/X -15..26 % at k >= 256, sorted rows -27 % at k = 1024, U/G/DG -1..4 %,
    // C3 -2.6 %.  Mode 1: a spread prologue of 16 evenly spaced chunks, then column
    // order; mode 0: column order.  Only the issuing lane walks the order
    // (incrementally, no divisions); the chunk id travels with the stage.
    const uint32_t nm = (uint32_t)nmine;
    uint32_t np = (nm >= 64u) ? 16u : nm / 4u;
    if ((order_mode & 3) == 0) np = 0;
    const uint32_t step = np ? nm / np : 1u;
    uint32_t pstride = 1;
    if ((order_mode & 3) == 2 && nm > 2u && lane == 0) {
        pstride = ((uint32_t)((double)nm * 0.6180339887498949)) | 1u;
        auto gcd = [](uint32_t a, uint32_t b) { while (b) { const uint32_t t = a % b; a = b; b = t; } return a; };
        while (gcd(pstride, nm) != 1u) pstride += 2;
    }
    uint32_t it_i = 0, it_blk = 0, it_off = 1, it_tail = np * step, it_p = 0;
    const uint32_t tailL = (uint32_t)(k + CH - 1) / CH + 1u;
    auto next_chunk = [&]() -> uint32_t {  // lane 0 only; chunk index relative to c_begin
        if ((order_mode & 3) == 3) {
            // the first chunk, the last L (enough for k: a descending row's smallest values),
            // then the rest in column order -- tied rows meet their smallest indices first
            if (nm <= tailL + 1u) return it_i++;
            if (it_i == 0u) return it_i++;
            if (it_i <= tailL) return nm - (it_i++);
            return 1u + (it_p++);
        }
        if ((order_mode & 3) == 2) {
            // the first and the last chunk first (they feed the starting bound: sorted rows,
            // ascending or descending, then start from their exact k-th when k <= 512),
            // then the strided permutation without those two
            if (it_i < 2u && nm > 2u) return (it_i++ == 0u) ? 0u : nm - 1u;
            uint32_t c;
            do {
                c = it_p;
                it_p += pstride;
                if (it_p >= nm) it_p -= nm;
            } while (nm > 2u && (c == 0u || c == nm - 1u));
            return c;
        }
        if (it_i < np) return (it_i++) * step;
        if (it_blk < np) {
            const uint32_t c = it_blk * step + it_off;
            if (++it_off == step) { it_off = 1; ++it_blk; }
            return c;
        }
        return it_tail++;
    };
    const uint32_t body_len = (uint32_t)(a1 - a0);  // < 2^31
    auto chunk_len = [&](uint32_t c) -> uint32_t { return min((uint32_t)CH, body_len - c * (uint32_t)CH); };
    auto issue = [&](int li) {
        const uint32_t c = (uint32_t)c_begin + next_chunk();
        const int st = li % S;
        cid[st] = c;
        const uint32_t bytes = chunk_len(c) * 4u;
        mbar_arrive_expect_tx(&mbar[st], bytes);
        bulk_g2s(ring + st * CH, dist + a0 + (uint64_t)c * CH, bytes, &mbar[st]);
    };

    if (lane == 0) {
        for (int s = 0; s < S; ++s) mbar_init(&mbar[s], 1);
        fence_mbar_init();
        for (int li = 0; li < S && li < nmine; ++li) issue(li);
    }
    if (WPR > 1 && wig == 0 && lane == 0) *grp_thr = 0xffffffffffffffffull;
    __syncwarp();
    if (WPR > 1) pool_group_bar(1 + grp, 32 * WPR);

    // ---- state ----------------------------------------------------------------------
    uint32_t Tk = kSentKey, Ti = kSentIdx;
    float tv = 0.f;
    bool fast = false;
    int n = 0;
    uint32_t bkey_r = kSentKey;  // the rigorous starting bound (kept for a failed speculation)
    bool spec_active = false;    // the bound in force is a speculative one, not yet verified

    auto tighten = [&](uint32_t kk, uint32_t ki) {
        if (pair_lt(kk, ki, Tk, Ti)) { Tk = kk; Ti = ki; }
        fast = Tk < 0xff800000u;
        tv = __uint_as_float(bits_of_key(Tk));
    };
    // pool full: exact k-th of everything seen so far becomes the threshold
    // Admission is loose (value <= bound value: one compare per element) until a
    // narrowing finds the k-th key tied across many pool entries; from then on this
    // warp uses the exact lexicographic test, which keeps tied rows (few distinct
    // values) from filling the pool with equal keys.
    bool exact_ties = (order_mode & 4) != 0;  // KSEL_LOOSE=1 experiment: exact from the start
    auto narrow = [&](uint32_t slack) {
        unsigned long long t;
        uint32_t ties = 0;
        if constexpr (Cfg::kPool <= 32 * 24) {
            // small pools: register-resident bisection (no histogram atomics)
            int nn;
            t = pool_narrow_regs<Cfg::kPool / 32>(pk, pi, n, (uint32_t)k, &nn, &ties, slack);
            n = nn;
        } else {
            t = pool_kth(pk, pi, n, (uint32_t)k, hist, &ties, slack);
            n = pool_compact(pk, pi, n, (uint32_t)(t >> 32), (uint32_t)t);
        }
        if (ties > 16u) exact_ties = true;
        const uint32_t kk = (uint32_t)(t >> 32), ki = (uint32_t)t;
        tighten(kk, ki);
        spec_active = false;  // (the pool's k-th: >= k seen pairs at or below the bound now)
        if (WPR > 1 && lane == 0) atomicMin(grp_thr, t);
    };
    // Exact path of one sub-step: the elements of this lane are the 4*G floats at
    // e(j) = ((g + j/4)*32 + lane)*4 + j%4 of the staged chunk `srcf` (x[j] in
    // registers).  Pre-filter again per element, run the exact lexicographic
    // test only on the flagged ones (re-read from shared memory), then append
    // the admitted pairs to the pool at warp-scanned positions.
    auto exact = [&](const float* srcf, uint32_t g, uint32_t len, uint32_t col0, const float(&x)[NS]) {
        uint32_t m = 0;
        if (fast) {
            // exact lexicographic admission, branch-free: value below the bound's, or
            // equal to it (same key; -0.0 == +0.0) with a smaller index.  Invalid slots of
            // a partial chunk hold +Inf and never pass.
            if (!exact_ties) {  // loose admission (x <= tv); ties are left to narrowing
#pragma unroll
                for (int j = 0; j < NS; ++j) m |= (uint32_t)(x[j] <= tv) << j;
            } else {
                const uint32_t cbase = col0 + (g * 32u + lane) * 4u;
#pragma unroll
                for (int j = 0; j < NS; ++j) {
                    const uint32_t col = cbase + (uint32_t)((j >> 2) * 128 + (j & 3));
                    m |= (uint32_t)(x[j] < tv || (x[j] == tv && col < Ti)) << j;
                }
            }
        } else {
#pragma unroll
            for (int u = 0; u < G; ++u)
                if (((g + (uint32_t)u) * 32u + lane) * 4u < len) m |= 0xfu << (4 * u);
        }
        auto elem = [&](int j) { return ((g + (uint32_t)(j >> 2)) * 32u + lane) * 4u + (uint32_t)(j & 3); };
        // The pool has room for a full sub-step after narrowing (P >= k' + 512); the
        // pairs flagged before a narrowing inside this sub-step are appended without a
        // re-test (harmless extra entries, dropped by the next narrowing).
        const uint32_t adm = m;
        uint32_t total;
        const uint32_t excl = warp_excl_scan(__popc(adm), lane, total);
        if (total == 0) return;
        if (n + (int)total > Cfg::kPool) {
            // stop the narrowing anywhere in [k, k + slack] pairs as long as this sub-step
            // still fits behind them (slack <= half the pool's spare room: 1/4 and 3/4
            // measured within 1 % on U/G, 1/2 -10..13 % on tied rows T/X at k = 128/256)
            const int room = Cfg::kPool - k - (int)total;
            narrow(room > 0 ? (uint32_t)min(room, (Cfg::kPool - k) / 2) : 0u);
        }
        int pos = n + (int)excl;
        for (uint32_t t = adm; t; t &= t - 1u) {
            const uint32_t e = elem(__ffs(t) - 1);
            pk[pos] = key_of(srcf[e]);
            pi[pos] = col0 + e;
            ++pos;
        }
        n += (int)total;
        __syncwarp();
    };

    // ---- unaligned head and tail (< 4 elements each; pool is empty, cannot overflow) ---------
    auto head_tail = [&]() {
        if (wig != 0) return;
        const uint32_t nh = (uint32_t)(a0 - g0), nt = (uint32_t)(g1 - a1);
        bool valid = false;
        uint64_t g = 0;
        if (lane < nh) { valid = true; g = g0 + lane; }
        else if (lane < nh + nt) { valid = true; g = a1 + (lane - nh); }
        const uint32_t bal = __ballot_sync(kFull, valid);
        if (valid) {
            const int pos = n + __popc(bal & lanemask_lt());
            pk[pos] = key_of(dist[g]);
            pi[pos] = (uint32_t)(g - g0);
        }
        n += __popc(bal);
        __syncwarp();
    };
    head_tail();

    // ---- starting bound: the k-th smallest key of the first S staged chunks -----------
    // (up to S*CH = 2048 values already in flight; bisection over their keys with
    // warp-wide counts).  At least k elements of the row are <= it, so
    // (key, largest index) bounds the k-th pair -- the stream then admits a few
    // times k candidates instead of everything until the pool first fills.
    constexpr int NB = Cfg::NB;
    if (nmine >= NB && !(order_mode & 32)) {
        uint32_t keys[NB * CH / 128 * 4];
        uint32_t nreal = 0;
#pragma unroll
        for (int li = 0; li < NB; ++li) {
            mbar_wait(&mbar[li], 0u);
            const uint32_t len = chunk_len(cid[li]);
            const float4* src4 = reinterpret_cast<const float4*>(ring + li * CH);
#pragma unroll
            for (int u = 0; u < CH / 128; ++u) {
                const uint32_t e4 = (uint32_t)u * 32u + lane;
                const bool ok = e4 * 4u < len;
                const float4 v = ok ? src4[e4] : make_float4(0.f, 0.f, 0.f, 0.f);
                const int base = (li * (CH / 128) + u) * 4;
                keys[base + 0] = ok ? key_of(v.x) : 0xffffffffu;
                keys[base + 1] = ok ? key_of(v.y) : 0xffffffffu;
                keys[base + 2] = ok ? key_of(v.z) : 0xffffffffu;
                keys[base + 3] = ok ? key_of(v.w) : 0xffffffffu;
                nreal += ok ? 4u : 0u;
            }
        }
        nreal = __reduce_add_sync(kFull, nreal);
        // Whether the speculative bound below will be used (k > 64 -- k' = 1024: k > 128 --
        // and sampled ranges that overlap): then the rigorous bisection is skipped (a failed
        // speculative share, ~1e-10, restarts cold).  C2 A/B (profiles/r02_c2_spec_k128_ab.txt):
        // k = 128 -2..-9 %, k = 64 mixed (+2 / -4 %), k = 32 +1..2 %: not below 65.
        // (k' < 1024 only: the k' = 1024 kernel, which never has a rigorous bound here
        // (k > NB * CH / 2), measured 3 % slower with this code shape -- it keeps the old one)
        bool spec_ok = false;
        uint32_t jj = 0;
        if (R < 32 && !(order_mode & 64) && k > 64 && nreal >= 64u) {
            uint32_t lo_max = 0u, hi_min = 0xffffffffu;
#pragma unroll
            for (int li = 0; li < NB; ++li) {
                uint32_t lo = 0xffffffffu, hi = 0u;
#pragma unroll
                for (int j = 0; j < CH / 128 * 4; ++j) {
                    const uint32_t kk2 = keys[li * (CH / 128) * 4 + j];
                    if (kk2 != 0xffffffffu) { lo = min(lo, kk2); hi = max(hi, kk2); }
                }
                lo_max = max(lo_max, __reduce_min_sync(kFull, lo));
                hi_min = min(hi_min, __reduce_max_sync(kFull, hi));
            }
            const uint64_t wlen = min((uint64_t)c_end * CH, (uint64_t)body_len) - (uint64_t)c_begin * CH;
            const double lam = (double)k * (double)nreal / (double)wlen;
            // (6 sigma as in the kNN filter: a failed share re-streams, and with ~2000 warps
            // per launch the slowest one sets the time -- measured with 3 sigma, P(fail) ~1e-3
            // per share: C2 U k = 256 0.103 -> 0.143 ms)
            jj = (uint32_t)ceil(lam + 6.0 * sqrt(lam) + 6.0);
            spec_ok = lo_max <= hi_min && jj < (uint32_t)k && jj < nreal;
        }
        if (!spec_ok && nreal >= (uint32_t)k && k <= NB * CH / 2) {
            // Bisection on the key bits below the common prefix of the smallest and
            // largest real key, stopped at bit kLow: the k-th key then lies in
            // [vkey, vkey + 2^kLow), so vkey | (2^kLow - 1) bounds it (>= k keys are
            // <= it; looser by < 2^-7 relative for floats, for about half the steps).
            constexpr int kLow = 16;
            uint32_t kmin = 0xffffffffu, kmax = 0u;
#pragma unroll
            for (int j = 0; j < NB * CH / 128 * 4; ++j) {
                kmin = min(kmin, keys[j]);  // (pads of a short chunk are 0xffffffff: only widen the range)
                kmax = max(kmax, keys[j]);
            }
            kmin = __reduce_min_sync(kFull, kmin);
            kmax = __reduce_max_sync(kFull, kmax);
            const int top = (kmin == kmax) ? -1 : 31 - __clz(kmin ^ kmax);
            uint32_t vkey = (top < 0) ? kmin : (kmin & ~((2u << top) - 1u));
            // (stops early at a candidate key with k..k + k/4 keys below it: any key with
            // >= k keys at or below it is a valid starting bound)
            uint32_t early = 0;
            const uint32_t kslack = (uint32_t)k + (uint32_t)k / 4u;
#pragma unroll 1
            for (int bit = top; bit >= kLow; --bit) {
                const uint32_t cand = vkey | (1u << bit);
                uint32_t c = 0;
#pragma unroll
                for (int j = 0; j < NB * CH / 128 * 4; ++j) c += (keys[j] < cand) ? 1u : 0u;
                c = __reduce_add_sync(kFull, c);
                if (c < (uint32_t)k) {
                    vkey = cand;
                } else if (c <= kslack) {
                    early = cand;
                    break;
                }
            }
            const uint32_t bkey = early ? early - 1u : (top >= kLow) ? (vkey | ((1u << kLow) - 1u)) : kmax;
            tighten(bkey, 0x7ffffffeu);
            bkey_r = bkey;
            if (WPR > 1 && lane == 0) atomicMin(grp_thr, ((unsigned long long)bkey << 32) | 0x7ffffffeu);
        }
        // Speculative bound (late r2; the kNN filter's idea, knn_fused.cu knn_spec_geometry):
        // the j-th smallest of the m sampled keys, j = lambda + 6 sqrt(lambda) + 6 with lambda
        // = k m / (this warp's element count).  On i.i.d. data the warp's count of keys <= it
        // is ~ (len / m) Gamma(j) >= k except with probability < 1e-10, so the stream admits
        // ~j len / m candidates instead of the ~k len / m of the rigorous bound (k-th of the
        // sample) and rarely narrows.  Verified at the end of the warp's share (>= k pool
        // pairs, or a narrowing / a group bound below it); otherwise the share is streamed
        // again from the rigorous bound.  Sampled chunks with disjoint key ranges (sorted
        // data: not a random sample) get no speculation.
        // (k > 128 only: measured on C2, speculation gains 7-46 % at k = 256 / 1024 and
        // costs 0-7 % at k <= 32 -- a few narrowings at most to save there)
        if (R == 32 && !(order_mode & 64) && k > 128 && nreal >= 64u) {
            uint32_t cmin[NB], cmax[NB];
#pragma unroll
            for (int li = 0; li < NB; ++li) {
                uint32_t lo = 0xffffffffu, hi = 0u;
#pragma unroll
                for (int j = 0; j < CH / 128 * 4; ++j) {
                    const uint32_t kk2 = keys[li * (CH / 128) * 4 + j];
                    if (kk2 != 0xffffffffu) { lo = min(lo, kk2); hi = max(hi, kk2); }
                }
                cmin[li] = __reduce_min_sync(kFull, lo);
                cmax[li] = __reduce_max_sync(kFull, hi);
            }
            uint32_t lo_max = 0u, hi_min = 0xffffffffu;
#pragma unroll
            for (int li = 0; li < NB; ++li) { lo_max = max(lo_max, cmin[li]); hi_min = min(hi_min, cmax[li]); }
            const uint64_t wlen = min((uint64_t)c_end * CH, (uint64_t)body_len) - (uint64_t)c_begin * CH;
            const double lam = (double)k * (double)nreal / (double)wlen;
            jj = (uint32_t)ceil(lam + 6.0 * sqrt(lam) + 6.0);
            spec_ok = lo_max <= hi_min && jj < (uint32_t)k && jj < nreal;
        }
        {
            if (spec_ok) {
                uint32_t kmin2 = 0xffffffffu, kmax2 = 0u;
#pragma unroll
                for (int j = 0; j < NB * CH / 128 * 4; ++j) {
                    kmin2 = min(kmin2, keys[j]);
                    kmax2 = max(kmax2, keys[j]);
                }
                kmin2 = __reduce_min_sync(kFull, kmin2);
                kmax2 = __reduce_max_sync(kFull, kmax2);
                constexpr int kLow = 16;
                const int top = (kmin2 == kmax2) ? -1 : 31 - __clz(kmin2 ^ kmax2);
                uint32_t vj = (top < 0) ? kmin2 : (kmin2 & ~((2u << top) - 1u));
#pragma unroll 1
                for (int bit = top; bit >= kLow; --bit) {
                    const uint32_t cand = vj | (1u << bit);
                    uint32_t c = 0;
#pragma unroll
                    for (int j = 0; j < NB * CH / 128 * 4; ++j) c += (keys[j] < cand) ? 1u : 0u;
                    c = __reduce_add_sync(kFull, c);
                    if (c < jj) vj = cand;
                }
                const uint32_t skey = (top >= kLow) ? (vj | ((1u << kLow) - 1u)) : kmax2;
                if (skey < Tk) {  // (the speculative pair (skey, 0x7ffffffe) below the bound in force)
                    tighten(skey, 0x7ffffffeu);
                    spec_active = true;
                }
            }
        }
    }

    // ---- streaming body ------------------------------------------------------------------
    // (pass 2, after a failed speculation, continues the ring's stage / barrier-phase
    // sequence: li runs on from nmine, so every mbarrier keeps its phase parity)
    int li0 = 0;
    for (;;) {
    for (int li = li0; li < li0 + nmine; ++li) {
        const int st = li % S;
        if (WPR > 1) {
            const unsigned long long sh = *reinterpret_cast<volatile unsigned long long*>(grp_thr);
            if (pair_lt((uint32_t)(sh >> 32), (uint32_t)sh, Tk, Ti)) spec_active = false;  // a verified bound takes over
            tighten((uint32_t)(sh >> 32), (uint32_t)sh);
        }
        // (a suspended wait: a warp whose data has not landed leaves its issue slots to
        // the other warps of the SM sub-partition instead of polling)
        mbar_wait_sleep(&mbar[st], (uint32_t)(li / S) & 1u);
        const uint32_t c = cid[st];
        const uint32_t len = chunk_len(c);
        const uint32_t col0 = (uint32_t)(a0 - g0) + c * (uint32_t)CH;
        const float* srcf = ring + st * CH;
        const float4* src = reinterpret_cast<const float4*>(srcf);
#pragma unroll 1
        for (int g = 0; g < CH / 128; g += G) {
            float x[NS];
            const float inf = __int_as_float(0x7f800000);  // never passes x <= tv in fast mode
            if (len == (uint32_t)CH) {  // (every chunk but a row's last: no per-element bounds)
#pragma unroll
                for (int u = 0; u < G; ++u) {
                    const float4 v = src[(uint32_t)(g + u) * 32u + lane];
                    x[4 * u + 0] = v.x;
                    x[4 * u + 1] = v.y;
                    x[4 * u + 2] = v.z;
                    x[4 * u + 3] = v.w;
                }
            } else {
#pragma unroll
                for (int u = 0; u < G; ++u) {
                    const uint32_t e4 = (uint32_t)(g + u) * 32u + lane;
                    const float4 v = (e4 * 4u < len) ? src[e4] : make_float4(inf, inf, inf, inf);
                    x[4 * u + 0] = v.x;
                    x[4 * u + 1] = v.y;
                    x[4 * u + 2] = v.z;
                    x[4 * u + 3] = v.w;
                }
            }
            bool go = true;
            if (fast) {
                // one compare per lane: the sub-step minimum (fminf skips NaN, which is never a
                // candidate).  Past the bound's index (col0 >= Ti) an element equal to the bound
                // value cannot precede the bound pair, so the test is strict: rows with heavy
                // ties then skip the sub-steps that only hold copies of the bound value.
                // (a tree, not a 15-deep chain: the sub-step is latency-bound when few warps run)
                // (3-input minima, FMNMX3 on sm_100: 10 instructions per 16 values instead of 15)
                static_assert(G == 4, "min tree shape");
                float gm[G];
#pragma unroll
                for (int u = 0; u < G; ++u) gm[u] = fminf(fmin3f(x[4 * u], x[4 * u + 1], x[4 * u + 2]), x[4 * u + 3]);
                const float mn = fminf(fmin3f(gm[0], gm[1], gm[2]), gm[3]);
                go = __any_sync(kFull, col0 >= Ti ? mn < tv : mn <= tv);
            }
            // The stage is refilled as soon as nothing reads it any more: right after the
            // vote when no lane has a candidate (the common case once the bound is tight:
            // every stage of the ring then stays in flight while the chunk is filtered),
            // else after the exact path, which re-reads admitted values from the stage.
            const bool last = g + G >= CH / 128;
            if (go && !(order_mode & 8)) exact(srcf, (uint32_t)g, len, col0, x);
            if (last) {
                __syncwarp();
                if (lane == 0 && li + S < li0 + nmine) issue(li + S);
            }
        }
    }

    if (!(spec_active && n < k)) break;
    // The speculative bound failed (fewer than k of this warp's pairs at or below it): stream
    // the share again from the rigorous bound (the ring is drained: every issued chunk was
    // consumed; the visit order restarts, the stage sequence continues).
    spec_active = false;
    n = 0;
    Tk = kSentKey;
    Ti = kSentIdx;
    fast = false;
    if (bkey_r != kSentKey) tighten(bkey_r, 0x7ffffffeu);
    __syncwarp();
    li0 = nmine;
    if (lane == 0) {
        it_i = 0; it_blk = 0; it_off = 1; it_tail = np * step; it_p = 0;
        for (int li = li0; li < li0 + S && li < li0 + nmine; ++li) issue(li);
    }
    __syncwarp();
    head_tail();
    }

    // ---- finish: exact top-k of this warp's share, sorted -----------------------------------
    if (order_mode & 16) {  // (phase-cost experiment: no final phase)
        if (lane == 0 && n == 0x7fffffff) out_val[row] = 0.f;
        return;
    }
    if (n > k) {
        const unsigned long long t = pool_kth(pk, pi, n, (uint32_t)k, hist);
        n = pool_compact(pk, pi, n, (uint32_t)(t >> 32), (uint32_t)t);
    }
    pool_sort<R>(pk, pi, n);

    if (WPR > 1) {
#pragma unroll 1
        for (int step = 1; step < WPR; step <<= 1) {
            pool_group_bar(1 + grp, 32 * WPR);
            if ((wig & (2 * step - 1)) == 0) {
                const uint32_t* ok2 = reinterpret_cast<const uint32_t*>(
                    smem + RPC * Cfg::kGroupBytes + (warp + step) * Cfg::kWarpStride + Cfg::kRingBytes);
                pool_merge_sorted<R>(pk, pi, ok2, ok2 + Cfg::kPool);
            }
        }
        if (wig != 0) return;
    }

    float* ov = out_val + row * (int64_t)k;
    int32_t* oi = out_idx + row * (int64_t)k;
    for (int e = (int)lane; e < k; e += 32) {
        const uint32_t key = pk[e];
        const uint32_t col = pi[e];
        const uint32_t bits = key_needs_regather(key) ? __float_as_uint(dist[g0 + col]) : bits_of_key(key);
        ov[e] = __uint_as_float(bits);
        oi[e] = (int32_t)(col + (uint32_t)coloff);
    }
}

template <int R, int WPR, int RPC, int SD>
static cudaError_t launch_pool_cfg(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi,
                                   SegMap seg, cudaStream_t stream) {
    using Cfg = PoolCfg<R, WPR, RPC, SD>;
    auto kern = ksel_pool_kernel<R, WPR, RPC, SD>;
    cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), Cfg::kSmem);
    if (e != cudaSuccess) return e;
    const int64_t grid = (Q + RPC - 1) / RPC;
    kern<<<(unsigned)grid, Cfg::kThreads, Cfg::kSmem, stream>>>(dist, Q, N, k, ov, oi, chunk_order_mode(), seg);
    note_launch();
    return cudaGetLastError();
}

// Largest configuration <= (WPR, RPC) whose shared memory fits one SM (227 KB):
// large queues with many warps per row fall back to fewer warps per CTA.
template <int R, int WPR, int RPC, int SD>
static cudaError_t launch_pool_fit(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi,
                                   SegMap seg, cudaStream_t stream) {
    if constexpr (PoolCfg<R, WPR, RPC, SD>::kSmem > kMaxSmemPerBlock) {
        if constexpr (RPC > 1) return launch_pool_fit<R, WPR, RPC / 2, SD>(dist, Q, N, k, ov, oi, seg, stream);
        else return launch_pool_fit<R, WPR / 2, 1, SD>(dist, Q, N, k, ov, oi, seg, stream);
    } else {
        return launch_pool_cfg<R, WPR, RPC, SD>(dist, Q, N, k, ov, oi, seg, stream);
    }
}

// wpr < 0 selects the deep ring (6 stages) with |wpr| warps per row.
template <int R>
cudaError_t launch_pool_r(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int wpr,
                          SegMap seg, cudaStream_t stream) {
    if (wpr < 0) {
        switch (-wpr) {
            case 1: return launch_pool_fit<R, 1, 1, 6>(dist, Q, N, k, ov, oi, seg, stream);
            case 2: return launch_pool_fit<R, 2, 1, 6>(dist, Q, N, k, ov, oi, seg, stream);
            case 4: return launch_pool_fit<R, 4, 1, 6>(dist, Q, N, k, ov, oi, seg, stream);
            default: return launch_pool_fit<R, 8, 1, 6>(dist, Q, N, k, ov, oi, seg, stream);
        }
    }
    switch (wpr) {
        case 1: return launch_pool_fit<R, 1, 1, 3>(dist, Q, N, k, ov, oi, seg, stream);
        case 2: return launch_pool_fit<R, 2, 1, 3>(dist, Q, N, k, ov, oi, seg, stream);
        case 4: return launch_pool_fit<R, 4, 1, 3>(dist, Q, N, k, ov, oi, seg, stream);
        default: return launch_pool_fit<R, 8, 1, 3>(dist, Q, N, k, ov, oi, seg, stream);
    }
}

// One object per queue size R (build.py compiles this file with -DKSEL_ONLY_R=R).
template cudaError_t launch_pool_r<KSEL_ONLY_R>(const float*, int64_t, int64_t, int, float*, int32_t*, int, SegMap,
                                                cudaStream_t);

}  // namespace ksel
