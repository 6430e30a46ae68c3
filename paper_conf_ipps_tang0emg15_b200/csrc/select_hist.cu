// KSEL_SPLIT_R
// select_hist.cu -- KSEL_ALGO_HIST (experiments library only): ksel_select with one
// CTA per row and a shared-memory candidate pool narrowed by range-adaptive radix
// histograms.  Bit-exact (tools/hist_check.py), but slower than the pool kernel on C2
// for U/G/DG/SA/SD at k <= 256 (profiles/r02_c2_hist_kernel_exp.txt), so not the product.
//
// Per row (8 filter warps + 1 producer warp, persistent over rows):
//   * the producer streams the CTA's rows in blocks of HS_HB = 2048 values with 1-D TMA
//     bulk copies into a HS_STAGES-deep ring (full/empty mbarriers), running ahead across
//     row boundaries; a row's last block is visited first (a descending row's smallest
//     values), then the others in column order;
//   * the first block is admitted whole; later values x are admitted iff (key(x), col) <
//     T, the k-th pair of the pool after its last narrowing (the Merge Queue's running
//     k-th threshold; the pool is the Buffered Search's candidate
//     buffer, L183-L187): one fp32 compare against a bound -- key < key(T) for blocks
//     after T's column, key <= key(T) for blocks before it -- behind a min per thread;
//   * the pool is narrowed to exactly k pairs once it holds k + 512 (and at the end):
//     Hierarchical Partition's discard-whole-groups step (L221-L231, value buckets as in
//     radix select [12]).  Each level bins the keys inside the current range [lo, lo +
//     width) into <= 2048 buckets of 2^s keys (s from the range, so keys sharing their top
//     bits still spread), keeps the bucket holding rank `want`, and stops once that bucket
//     is taken whole; a single key holding the rank is resolved by the same levels over
//     the columns (reading R1);
//   * warp 0 sorts the k pairs in registers (bitonic network) and emits them, -0.0 / NaN
//     bits re-read from the row.
#include <cstdint>
#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_common.cuh"
#include "ksel_internal.h"

#ifndef KSEL_ONLY_R
#error "compile once per queue size with -DKSEL_ONLY_R=1|2|4|8|16|32"
#endif
#ifdef KSEL_EXPERIMENTS  // (not in the product library: see dispatch.cu)

namespace ksel {

constexpr int HS_THREADS = 256;
constexpr int HS_WARPS = HS_THREADS / 32;
constexpr int HS_HB = 2048;                       // values per block (8 KB, 2 float4 per thread)
constexpr int HS_V4 = HS_HB / 4 / HS_THREADS;     // float4 per thread per block
static_assert(HS_V4 == 2, "append select tree assumes 2 float4 per thread");
constexpr int HS_STAGES = 4;                      // ring: 32 KB of the row stream in flight per CTA
constexpr int HS_BINS = 2048;
constexpr int HS_CAP = 4096;                      // pool pairs
constexpr int HS_NARROW_AT = HS_CAP - HS_HB - 8;  // narrow when the pool holds more (room: a block + tail)
// 3 CTAs per SM (96 KB of the stream in flight) while the final register sort is small
__host__ __device__ constexpr int hs_ctas_per_sm(int R) { return R <= 8 ? 3 : 2; }
static_assert(HS_NARROW_AT >= KSEL_MAX_K, "pool too small for k");

struct HistSmem {
    float ring[HS_STAGES][HS_HB];
    unsigned long long pool[HS_CAP];
    union {
        uint32_t hist[HS_BINS];
        unsigned long long keep[HS_BINS / 2];  // compaction side buffer (k <= 1024 pairs)
    };
    uint64_t full[HS_STAGES];   // block landed (1 arrival + bytes)
    uint64_t empty[HS_STAGES];  // stage read by the HS_WARPS filter warps
    uint32_t wsum[HS_WARPS];
    uint32_t red[4];
    uint32_t res[3];
    int count;
    int kept;
};
static_assert(HS_BINS / 2 >= KSEL_MAX_K, "side buffer too small for k");

// Consumer-only barriers (named barrier 1: the HS_THREADS filter threads; the producer
// warp never joins).
static __device__ __forceinline__ void cbar() {
    asm volatile("bar.sync 1, %0;" ::"r"(HS_THREADS) : "memory");
}
static __device__ __forceinline__ bool cbar_or(bool pred) {
    uint32_t r;
    asm volatile(
        "{\n\t.reg .pred p, q;\n\tsetp.ne.u32 p, %1, 0;\n\t"
        "barrier.cta.red.or.pred q, 1, %2, p;\n\tselp.u32 %0, 1, 0, q;\n\t}"
        : "=r"(r)
        : "r"((uint32_t)pred), "r"(HS_THREADS)
        : "memory");
    return r != 0;
}

// Row geometry: a scalar head up to 16-byte alignment, nb4 float4s in blocks of HS_HB
// values, a scalar tail.
struct HsRow {
    const float* rp;
    int64_t head, nb4, nblk;
};
static __device__ __forceinline__ HsRow hs_row(const float* dist, int64_t row, int64_t N) {
    HsRow g;
    g.rp = dist + row * N;
    const int64_t mis = (int64_t)(((16u - (reinterpret_cast<uintptr_t>(g.rp) & 15u)) & 15u) >> 2);
    g.head = mis < N ? mis : N;
    g.nb4 = (N - g.head) >> 2;
    g.nblk = (g.nb4 + HS_HB / 4 - 1) / (HS_HB / 4);
    return g;
}
// Visit order of a row's blocks: the last first (a descending row's smallest values),
// then the rest in column order.
static __device__ __forceinline__ int64_t hs_blk(int64_t j, int64_t nblk) { return j == 0 ? nblk - 1 : j - 1; }

// Block exclusive scan of one value per thread; the total in *tot.
static __device__ __forceinline__ uint32_t hs_block_scan(uint32_t v, uint32_t* wsum, uint32_t* tot) {
    const uint32_t lane = lane_id();
    const int warp = threadIdx.x >> 5;
    uint32_t inc = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, inc, d);
        if (lane >= (uint32_t)d) inc += t;
    }
    if (lane == 31) wsum[warp] = inc;
    cbar();
    uint32_t before = 0, all = 0;
#pragma unroll
    for (int w = 0; w < HS_WARPS; ++w) {
        const uint32_t s = wsum[w];
        before += (w < warp) ? s : 0u;
        all += s;
    }
    cbar();  // wsum reusable
    *tot = all;
    return before + inc - v;
}

static __device__ __forceinline__ int bits_needed(uint64_t x) { return x ? 64 - __clzll((long long)x) : 0; }

// Histogram levels over one 32-bit field of the pool entries that pass `member`: on
// entry every member's field lies in [lo, lo + width) and `want` (1-based) is a rank
// among the members; on exit [lo, lo + width) is the range holding that rank, `want`
// its rank inside it.  Returns true when the range is taken whole (its population is
// `want`), else width == 1.
template <class Field, class Member>
static __device__ bool hs_levels(HistSmem& sm, int n, Field field, Member member, uint32_t& lo, uint64_t& width,
                          uint32_t& want) {
    const int tid = threadIdx.x;
    const uint32_t lane = lane_id();
    for (;;) {
        const int nb = bits_needed(width - 1);
        const int s = nb > 11 ? nb - 11 : 0;
        for (int b = tid; b < HS_BINS; b += HS_THREADS) sm.hist[b] = 0u;
        cbar();
        for (int base = 0; base < n; base += HS_THREADS) {
            const int e = base + tid;
            bool in = false;
            uint32_t d = 0xffffffffu;
            if (e < n) {
                const unsigned long long c = sm.pool[e];
                const uint32_t f = field(c);
                in = member(c) && f >= lo && (uint64_t)(f - lo) < width;
                if (in) d = (f - lo) >> s;
            }
            // lanes with the same bucket add once (ties would serialise the atomics)
            const uint32_t same = __match_any_sync(kFull, d);
            if (in && lane == (uint32_t)(__ffs(same) - 1)) atomicAdd(&sm.hist[d], (uint32_t)__popc(same));
        }
        cbar();
        uint32_t h[HS_BINS / HS_THREADS], tsum = 0;
#pragma unroll
        for (int j = 0; j < HS_BINS / HS_THREADS; ++j) {
            h[j] = sm.hist[tid * (HS_BINS / HS_THREADS) + j];
            tsum += h[j];
        }
        uint32_t tot;
        const uint32_t excl = hs_block_scan(tsum, sm.wsum, &tot);
        if (excl < want && want <= excl + tsum) {
            uint32_t acc = excl;
#pragma unroll
            for (int j = 0; j < HS_BINS / HS_THREADS; ++j) {
                if (acc < want && want <= acc + h[j]) {
                    sm.res[0] = (uint32_t)(tid * (HS_BINS / HS_THREADS) + j);
                    sm.res[1] = acc;
                    sm.res[2] = h[j];
                }
                acc += h[j];
            }
        }
        cbar();
        const uint32_t b = sm.res[0], before = sm.res[1], pop = sm.res[2];
        cbar();  // res reusable
        want -= before;
        lo += b << s;
        const uint64_t rest = width - ((uint64_t)b << s);
        width = rest < (1ull << s) ? rest : (1ull << s);
        if (pop == want) return true;
        if (width == 1) return false;
    }
}

// Narrow the pool (sm.count > k pairs, no appends in flight) to its k smallest; returns
// the largest kept pair.
static __device__ unsigned long long hs_narrow(HistSmem& sm, int k) {
    const int tid = threadIdx.x;
    const uint32_t lane = lane_id();
    // key range of the pool
    if (tid == 0) {
        sm.red[0] = 0xffffffffu;
        sm.red[1] = 0u;
        sm.kept = 0;
    }
    cbar();
    const int n = sm.count;
    uint32_t mn = 0xffffffffu, mx = 0u;
    for (int e = tid; e < n; e += HS_THREADS) {
        const uint32_t key = (uint32_t)(sm.pool[e] >> 32);
        mn = min(mn, key);
        mx = max(mx, key);
    }
    mn = __reduce_min_sync(kFull, mn);
    mx = __reduce_max_sync(kFull, mx);
    if (lane == 0) {
        atomicMin(&sm.red[0], mn);
        atomicMax(&sm.red[1], mx);
    }
    cbar();
    uint32_t lo = sm.red[0];
    uint64_t width = (uint64_t)sm.red[1] - lo + 1u;
    uint32_t want = (uint32_t)k;
    cbar();  // red reusable
    const bool whole = hs_levels(
        sm, n, [](unsigned long long c) { return (uint32_t)(c >> 32); }, [](unsigned long long) { return true; },
        lo, width, want);
    unsigned long long incl;  // keep the pairs c <= incl
    if (whole) {
        const uint64_t hi = (uint64_t)lo + width;  // exclusive key bound, <= 2^32
        incl = (hi >= (1ull << 32)) ? ~0ull : ((hi << 32) - 1u);
    } else {
        // one key v holds rank `want` among its ties: resolve by column
        const uint32_t v = lo;
        if (tid == 0) {
            sm.red[2] = 0xffffffffu;
            sm.red[3] = 0u;
        }
        cbar();
        uint32_t imn = 0xffffffffu, imx = 0u;
        for (int e = tid; e < n; e += HS_THREADS) {
            const unsigned long long c = sm.pool[e];
            if ((uint32_t)(c >> 32) == v) {
                imn = min(imn, (uint32_t)c);
                imx = max(imx, (uint32_t)c);
            }
        }
        imn = __reduce_min_sync(kFull, imn);
        imx = __reduce_max_sync(kFull, imx);
        if (lane == 0) {
            atomicMin(&sm.red[2], imn);
            atomicMax(&sm.red[3], imx);
        }
        cbar();
        uint32_t ilo = sm.red[2];
        uint64_t iw = (uint64_t)sm.red[3] - ilo + 1u;
        cbar();
        hs_levels(
            sm, n, [](unsigned long long c) { return (uint32_t)c; },
            [v](unsigned long long c) { return (uint32_t)(c >> 32) == v; }, ilo, iw, want);
        incl = ((unsigned long long)v << 32) | (uint64_t)(ilo + (uint32_t)iw - 1u);
    }
    // compact the k kept pairs through the side buffer
    unsigned long long tmax = 0ull;
    for (int base = 0; base < n; base += HS_THREADS) {
        const int e = base + tid;
        unsigned long long c = 0ull;
        bool keep = false;
        if (e < n) {
            c = sm.pool[e];
            keep = c <= incl;
        }
        const uint32_t m = __ballot_sync(kFull, keep);
        int pos = 0;
        if (lane == 0 && m) pos = atomicAdd(&sm.kept, __popc(m));
        pos = __shfl_sync(kFull, pos, 0);
        if (keep) {
            sm.keep[pos + __popc(m & lanemask_lt())] = c;
            tmax = c > tmax ? c : tmax;
        }
    }
    cbar();
    for (int e = tid; e < k; e += HS_THREADS) sm.pool[e] = sm.keep[e];
#pragma unroll
    for (int d = 16; d; d >>= 1) {
        const unsigned long long o = __shfl_xor_sync(kFull, tmax, d);
        tmax = o > tmax ? o : tmax;
    }
    cbar();  // keep[] read
    if (lane == 0) sm.keep[tid >> 5] = tmax;
    if (tid == 0) sm.count = k;
    cbar();
    unsigned long long T = 0ull;
#pragma unroll
    for (int w = 0; w < HS_WARPS; ++w) T = sm.keep[w] > T ? sm.keep[w] : T;
    cbar();
    return T;
}

// fp32 bound t with  key(x) < kT  <=>  x <= t  for every non-NaN x; NaN (the largest
// key) is then admitted only by no bound, as no key lies above it.
static __device__ __forceinline__ float hs_bound(uint32_t kT) {
    if (kT > 0xff800000u) return __int_as_float(0x7f800000);  // T is NaN: every non-NaN value
    if (kT <= 0x007fffffu) return __int_as_float(0x7fc00000);  // T is -Inf: nothing (x <= NaN)
    uint32_t kb = kT - 1u;
    if (kb == 0x7fffffffu) kb = 0x7ffffffeu;  // T is +-0: -0.0 shares +0.0's key, bound below both
    return __uint_as_float(bits_of_key(kb));
}

static __device__ __forceinline__ float hs_comp(const float4& q, int c) {
    return c == 0 ? q.x : c == 1 ? q.y : c == 2 ? q.z : q.w;
}

template <int R>
__global__ void __launch_bounds__(HS_THREADS + 32, hs_ctas_per_sm(R))
    ksel_hist_kernel(const float* __restrict__ dist, int64_t Q, int64_t N, int k, int narrow_at,
                     float* __restrict__ out_val, int32_t* __restrict__ out_idx) {
    extern __shared__ __align__(128) uint8_t smem_raw[];
    HistSmem& sm = *reinterpret_cast<HistSmem*>(smem_raw);
    const int tid = threadIdx.x;
    const uint32_t lane = lane_id();

    if (tid == 0) {
        for (int st = 0; st < HS_STAGES; ++st) {
            mbar_init(&sm.full[st], 1);
            mbar_init(&sm.empty[st], HS_WARPS);
        }
        fence_mbar_init();
    }
    __syncthreads();
    if (tid >= HS_THREADS) {
        // ---- producer warp (one lane): the CTA's blocks, row after row, into the ring ----
        if (tid == HS_THREADS) {
            uint32_t li = 0;
            for (int64_t row = blockIdx.x; row < Q; row += gridDim.x) {
                const HsRow g = hs_row(dist, row, N);
                for (int64_t j = 0; j < g.nblk; ++j, ++li) {
                    const int st = (int)(li % HS_STAGES);
                    if (li >= (uint32_t)HS_STAGES) mbar_wait_sleep(&sm.empty[st], ((li / HS_STAGES) - 1u) & 1u);
                    const int64_t v0 = hs_blk(j, g.nblk) * HS_HB, len = min((int64_t)HS_HB, 4 * g.nb4 - v0);
                    mbar_arrive_expect_tx(&sm.full[st], (uint32_t)len * 4u);
                    bulk_g2s(sm.ring[st], g.rp + g.head + v0, (uint32_t)len * 4u, &sm.full[st]);
                }
            }
        }
        return;
    }

    uint32_t li = 0;  // blocks consumed by this CTA
    for (int64_t row = blockIdx.x; row < Q; row += gridDim.x) {
        const HsRow g = hs_row(dist, row, N);
        const float* rp = g.rp;
        const int64_t tail0 = g.head + 4 * g.nb4;

        if (tid == 0) sm.count = 0;
        cbar();
        // append this thread's admitted values (bit 4j + c of m: component c of v[j]);
        // my_end: the pool size just after this thread's (or its warp's) last append --
        // its maximum over the CTA is the pool size, reduced by the block barrier
        // (sm.count itself may already hold the next block's appends of faster warps)
        int my_end = 0;
        auto append = [&](const float4* v, uint32_t m, uint32_t col_base) {
            if (!m) return;
            const int cnt = __popc(m);
            int p = atomicAdd(&sm.count, cnt);
            my_end = max(my_end, p + cnt);
            if (m == (1u << (4 * HS_V4)) - 1u) {  // the whole slice
#pragma unroll
                for (int j = 0; j < HS_V4; ++j) {
                    const uint32_t col0 = col_base + 4u * (uint32_t)(j * HS_THREADS + tid);
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        sm.pool[p + 4 * j + c] = ((unsigned long long)key_of(hs_comp(v[j], c)) << 32) | (col0 + c);
                }
            } else {
                while (m) {  // set bits only; the value through a select tree (no local copy)
                    const int j = __ffs(m) - 1;
                    m &= m - 1u;
                    const float4 q = (j >> 2) == 0 ? v[0] : v[HS_V4 - 1];
                    const float x = (j & 2) ? ((j & 1) ? q.w : q.z) : ((j & 1) ? q.y : q.x);
                    const uint32_t col = col_base + 4u * (uint32_t)((j >> 2) * HS_THREADS + tid) + (uint32_t)(j & 3);
                    sm.pool[p++] = ((unsigned long long)key_of(x) << 32) | col;
                }
            }
        };
        // head (< 4 values, before every block in column order): admitted
        if (tid < g.head) {
            const int p = atomicAdd(&sm.count, 1);
            sm.pool[p] = ((unsigned long long)key_of(rp[tid]) << 32) | (uint32_t)tid;
            my_end = p + 1;
        }
        // threshold T = (kT, iT) once the pool was narrowed; bounds for later blocks:
        // columns above iT admit key < kT (x <= t_lt), columns below admit key <= kT
        // (x <= t_le; every value when kT is NaN's key)
        bool has_t = false;
        uint32_t kT = 0, iT = 0;
        float t_lt = 0.f, t_le = 0.f;
        const int nblk = (int)g.nblk, nv = (int)(4 * g.nb4);
        for (int j = 0; j < nblk; ++j, ++li) {
            const int st = (int)(li % HS_STAGES);
            const int v0 = (j == 0 ? nblk - 1 : j - 1) * HS_HB;  // hs_blk
            const int len = min(HS_HB, nv - v0);
            const uint32_t col_base = (uint32_t)g.head + (uint32_t)v0;
            mbar_wait(&sm.full[st], (li / HS_STAGES) & 1u);
            float4 cur[HS_V4];
            const float4* src = reinterpret_cast<const float4*>(sm.ring[st]);
#pragma unroll
            for (int q = 0; q < HS_V4; ++q) cur[q] = src[q * HS_THREADS + tid];
            __syncwarp();
            if (lane == 0) mbar_arrive_cta(&sm.empty[st]);  // this warp's slice is in registers
            uint32_t valid = (1u << (4 * HS_V4)) - 1u;
            if (len < HS_HB) {  // a row's partial block: stale ring words become NaN (never admitted)
#pragma unroll
                for (int q = 0; q < HS_V4; ++q) {
                    if (4 * (q * HS_THREADS + tid) >= len) {
                        valid &= ~(0xfu << (4 * q));
                        cur[q] = make_float4(__int_as_float(0x7fc00000), __int_as_float(0x7fc00000),
                                             __int_as_float(0x7fc00000), __int_as_float(0x7fc00000));
                    }
                }
            }
            const bool below = has_t && col_base + (uint32_t)len <= iT;  // every column < iT
            if (!has_t || (below && kT == 0xffffffffu)) {  // every value (NaN included)
                append(cur, valid, col_base);
            } else {
                const float t = below ? t_le : t_lt;
                float mn = fminf(fminf(cur[0].x, cur[0].y), fminf(cur[0].z, cur[0].w));
#pragma unroll
                for (int q = 1; q < HS_V4; ++q) mn = fminf(mn, fminf(fminf(cur[q].x, cur[q].y), fminf(cur[q].z, cur[q].w)));
                if (mn <= t) {
                    uint32_t m = 0;
#pragma unroll
                    for (int q = 0; q < HS_V4; ++q) {
                        m |= (cur[q].x <= t ? 1u : 0u) << (4 * q);
                        m |= (cur[q].y <= t ? 2u : 0u) << (4 * q);
                        m |= (cur[q].z <= t ? 4u : 0u) << (4 * q);
                        m |= (cur[q].w <= t ? 8u : 0u) << (4 * q);
                    }
                    append(cur, m, col_base);
                }
            }
            // stage st read, pool appends visible; narrow when the pool outgrew its limit
            // (before the first narrowing: k, while blocks remain)
            const int lim = has_t ? narrow_at : k;
            const bool narrow = cbar_or(my_end > lim) && (has_t || j + 1 < nblk);
            if (narrow) {
                const unsigned long long T = hs_narrow(sm, k);
                my_end = 0;
                has_t = true;
                kT = (uint32_t)(T >> 32);
                iT = (uint32_t)T;
                t_lt = hs_bound(kT);
                t_le = __uint_as_float(bits_of_key(kT));  // (kT = NaN's key: unused)
            }
        }
        // tail (< 4 values, after every block): admitted
        if (tid < N - tail0) {
            const int p = atomicAdd(&sm.count, 1);
            sm.pool[p] = ((unsigned long long)key_of(rp[tail0 + tid]) << 32) | (uint32_t)(tail0 + tid);
        }
        cbar();
        const int n = sm.count;
        if (n > k) hs_narrow(sm, k);
        // sort the k pairs ascending (warp 0, registers) and emit
        if (tid < 32) {
            WArr<R> a;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int e = r * 32 + (int)lane;
                const unsigned long long c = e < k ? sm.pool[e] : ((unsigned long long)kSentKey << 32 | kSentIdx);
                a.k[r] = (uint32_t)(c >> 32);
                a.i[r] = (uint32_t)c;
            }
            warr_sort<R>(a, lane);
            float* ov = out_val + row * (int64_t)k;
            int32_t* oi = out_idx + row * (int64_t)k;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int e = r * 32 + (int)lane;
                if (e < k) {
                    ov[e] = __uint_as_float(key_needs_regather(a.k[r]) ? __float_as_uint(rp[a.i[r]])
                                                                       : bits_of_key(a.k[r]));
                    oi[e] = (int32_t)a.i[r];
                }
            }
        }
        cbar();
    }
}

template <int R>
cudaError_t launch_hist_r(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi, int sms,
                          cudaStream_t stream) {
    auto kern = ksel_hist_kernel<R>;
    const int smem = (int)sizeof(HistSmem);
    cudaError_t e = ensure_smem_attr(reinterpret_cast<const void*>(kern), smem);
    if (e != cudaSuccess) return e;
    // narrow once the pool holds `slack` pairs beyond k: a tighter threshold sooner
    // (fewer admissions) against more narrowings
    int slack = 512;
#ifdef KSEL_EXPERIMENTS
    slack = env_int("KSEL_HIST_SLACK", slack);
#endif
    const int narrow_at = (k + slack < HS_NARROW_AT) ? k + slack : HS_NARROW_AT;
    const int64_t slots = (int64_t)hs_ctas_per_sm(R) * sms;
    const int64_t grid = Q < slots ? Q : slots;
    kern<<<(unsigned)grid, HS_THREADS + 32, smem, stream>>>(dist, Q, N, k, narrow_at, ov, oi);
    note_launch();
    return cudaGetLastError();
}

template cudaError_t launch_hist_r<KSEL_ONLY_R>(const float*, int64_t, int64_t, int, float*, int32_t*, int,
                                                cudaStream_t);

}  // namespace ksel
#endif  // KSEL_EXPERIMENTS
