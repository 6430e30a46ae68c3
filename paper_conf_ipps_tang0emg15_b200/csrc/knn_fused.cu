// knn_fused.cu -- knn_search: tcgen05/TMEM distance FILTER fused with k-selection,
// followed by exact rescoring of the survivors (knn_rescore.cu).
//
// The k-NN of the paper has two phases (Sec. II.A): Euclidean
// distances between every query and reference, then k-selection over each
// query's row of N distances.  The paper computes the Q x N matrix with "the
// method of [3]" and stores it in global memory (L243); here the matrix never
// exists.  d~(q, r) = |q|^2 + |r|^2 - 2 q.r (reading R9: squared L2), with the dot
// products on the 5th-gen tensor cores:
//
//   * points are centred (x' = x - c, c a rounded sample mean) and each tile scaled by a
//     power of two, then rounded to fp16 once: ONE kind::f16 MMA pass (fp16 x fp16 ->
//     fp32 TMEM accumulator); the error of that rounding is in the bound eps_q below.
//   * the norms ride in the same accumulation: A holds -2 s_q q' and one extra
//     16-wide bf16 K block [s n1, s n2, s n3, s, s, s, 0...] with |q'|^2 = n1+n2+n3 split
//     three ways (24 significant bits), B holds [s, s, s, s m1, s m2, s m3, 0...] for
//     |r'|^2 -- so the accumulator IS s_q s_t d~(q, r) and the epilogue touches each
//     distance once (it compares against the bound scaled the same way).
//   * d~ only FILTERS: |d~ - d| <= eps_q (a rigorous bound, knn_common.cuh knn_eps,
//     DESIGN.md reading R21, ~0.4 % of the k-th distance on the paper's workload), so a
//     reference can be in the exact top-k only if d~ <= T + 2 eps_q for any k-th
//     value T of d~ over k references; the epilogue admits exactly those, pools keep
//     that band above their k-th d~, and knn_rescore.cu recomputes every survivor in
//     the oracle's own arithmetic and selects the exact top-k -- bit-identical to the
//     CPU oracle.  A query whose band overflows its pool (massive ties of d~, or
//     non-finite input) is flagged and solved by an exact brute-force fallback.
//   * CTA = one tile of 128 queries (TMEM lanes, A operand resident in shared
//     memory) x a contiguous range of 256-reference tiles (TMEM columns, B
//     operand streamed by 1-D TMA bulk copies from a pre-tiled image);
//     warp 0 = producer, warp 1 = TMEM allocator + single-thread MMA issuer,
//     warps 2-17 = epilogue (four per TMEM lane quadrant; one thread per query: the
//     paper's thread-per-query layout, L243), double-buffered 2 x 256-column accumulators.
//   * a speculative pre-pass of the same kernel over a strided sample of reference tiles
//     gives each query a starting bound T_spec (verified later in knn_rescore.cu).
//   * epilogue: tcgen05.ld 32 columns at a time, an fp32 min/vote pre-filter against
//     the running bound plus the band, a rare path that appends packed
//     (key(d~) << 32 | index) pairs to a per-query pool in global memory,
//     warp-cooperative narrowing (register bisection, radix select for large pools)
//     when a pool fills; the k-th pair of every narrowing is published per query
//     (atomicMin) so all splits share bounds.
//   * queries are processed in chunks so that the pools stay below 2 GiB.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_common.cuh"
#include "ksel_internal.h"
#include "ksel_pool.cuh"
#include "knn_common.cuh"

namespace ksel {

constexpr int KNN_BM = 128;                              // queries per tile (TMEM lanes)
constexpr int KNN_BN = 256;                              // references per tile (accumulator columns)
constexpr int KNN_KS = 32;                               // dims per pipeline stage
constexpr int KNN_NORM_A_BYTES = 16 * KNN_BM * 2;         // norm block of a query tile
// epilogue warps EW: 4 (one per TMEM lane quadrant, all 256 columns of a tile) or
// 8 (two per quadrant, 128 columns each); + producer + MMA issuer
constexpr int KNN_MAX_EW = 16;
__host__ __device__ constexpr int knn_threads(int ew) { return 64 + 32 * ew; }
constexpr int KNN_SB = 32;                                // sampling histogram buckets
constexpr int KNN_CW = 64;                                // accumulator columns per epilogue step
constexpr int kNarrowRegs = 40;  // register-resident narrowing: pools of <= 1280 pairs
constexpr unsigned long long kSentPair = ((unsigned long long)kSentKey << 32) | kSentIdx;

struct KnnGeom {
    int64_t N, Q;
    int D, Dp, KS;       // dims, padded dims (multiple of 32), stages per tile
    int NT, QT, S;       // ref tiles, query tiles, reference splits
    int k, P;            // k, per-query pool capacity
    int NS;              // ring stages
    int64_t idx_offset;
    int ntiles, tstride; // this launch visits reference tiles i * tstride, i < ntiles (split over S)
    int sample_tiles;    // cold CTAs (blockIdx < sample_ctas) first histogram this many tiles
    int sample_ctas;
    int halves;          // column halves per tile (EW / 4): pools per split
    int pcap;            // pool fill that triggers a narrowing before a tile (<= P)
    int nstride;         // tiles between two bound refreshes / narrowing checks (room: nstride x BN)
    int spec_ms;         // speculative pre-pass: sampled tiles (0: none)
    int prepass;         // this launch IS the pre-pass: a query whose band overflows is not
                         // failed (it merely gets a looser T_spec); qthr = the T_spec output
    int cs;              // cluster size: CTAs (consecutive query tiles, same reference range) that
                         // share every reference stage through one multicast load
    int QTp;             // query tiles padded to a multiple of cs (padding tiles select nothing)
    int cold_splits;     // leading splits run by first-wave CTAs (no published bound yet)
    int cold_w;          // their share of the reference tiles relative to the others (per mille)
    // first logical tile of split s: split s weighs cold_w / 1000 if s < cold_splits, else 1
    __host__ __device__ int split_begin(int s) const {
        auto W = [&](int x) -> int64_t {
            const int c = x < cold_splits ? x : cold_splits;
            return (int64_t)c * cold_w + (int64_t)(x - c) * 1000;
        };
        return (int)((int64_t)ntiles * W(s) / W(S));
    }
    int BN;              // references per tile (accumulator columns): 256, or 128 with QPC = 2
    int QPC;             // query tiles per CTA sharing every reference stage (1 or 2)
    int EW;              // epilogue warps of the launch (4, or 8)
    __host__ __device__ int stage_bytes() const { return KNN_KS * BN * 2; }  // fp16
    __host__ __device__ int norm_b_bytes() const { return 16 * BN * 2; }
    __host__ __device__ size_t tile_bytes() const { return (size_t)KS * stage_bytes() + norm_b_bytes(); }
    __host__ __device__ int a_bytes() const { return Dp * 256 + KNN_NORM_A_BYTES; }
};

// ---------------------------------------------------------------------------
// prologue: centred, per-tile scaled fp16 operands in the UMMA canonical
// (K-major, no-swizzle) image
// ---------------------------------------------------------------------------
// Core matrix = 8 rows x 16 bytes (8 halves along K), rows 16 B apart; 8-row
// groups 128 B apart (SBO); 8-element K chunks ROWS*16 B apart (LBO).
//   ref image : [tile][stage][4 chunks][256 rows][8] fp16 (16 KB per stage), then the
//               tile's bf16 norm block [2 chunks][256 rows][8]
//   query img : [tile][Dp/8 chunks][128 rows][8] fp16, then the bf16 norm block
//
// Distances are translation invariant: every point is first centred, x' = fl(x - c)
// with c the mean of a reference sample (knn_center_kernel), which shrinks |x'| and
// with it every term of the error bound (U[0,1]^128: |x|^2 ~ 43 -> |x'|^2 ~ 11).  Each
// tile (256 references / 128 queries) is then scaled by a power of two sigma so that its
// largest magnitude lands in [2^14, 2^15) (queries: of -2 sigma x'), and rounded to
// fp16 once -- one kind::f16 MMA pass instead of bf16 hi/lo x 3.  The accumulator holds
// sigma_q sigma_t d~; the epilogue compares it with the bound scaled the same way and
// unscales (exactly, powers of two) only the candidates it keeps.

// bf16 pair of two floats (round to nearest even)
__device__ __forceinline__ uint32_t bf2(float a, float b) {
    return (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(a)) |
           ((uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn(b)) << 16);
}
__device__ __forceinline__ uint32_t h2(float a, float b) {
    return (uint32_t)__half_as_ushort(__float2half_rn(a)) | ((uint32_t)__half_as_ushort(__float2half_rn(b)) << 16);
}

// c[d] = the mean of a strided sample of <= 16384 reference rows, rounded to a multiple of
// 2^(ilogb(sd_d) - 4) (sd_d the sample's spread in dim d): any c is exact (it only has to
// make |x'| small), and a coarse c keeps x' = x - c exact for integer-valued data (then
// every fp16 operand is exact).  c = 0 for the padding dims.  knn_sum_kernel: block
// (x, y) adds dims [32x, 32x + 32) of rows y*8 + warp + 256 i of the sample into csum
// (double atomics; [2][Dp]: sums, sums of squares; then [2][Dp] u32: the sample's min and
// max per dim as order keys, min stored inverted so that both are atomicMax from 0);
// knn_center_value turns them into c, knn_sample_range into the largest |x - c| sampled.
__global__ void __launch_bounds__(256)
    knn_sum_kernel(const float* __restrict__ ref, int64_t N, int D, int Dp, double* __restrict__ csum) {
    __shared__ double part[2][8][33];
    __shared__ uint32_t pk[2][8][33];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int d = blockIdx.x * 32 + lane;
    const int64_t ns = N < 16384 ? N : 16384;
    const int64_t stride = N / ns;
    double s = 0.0, s2 = 0.0;
    uint32_t kmn = 0u, kmx = 0u;  // (inverted min key, max key)
    if (d < D)
        for (int64_t i = (int64_t)blockIdx.y * 8 + warp; i < ns; i += 8 * (int64_t)gridDim.y) {
            const float f = __ldg(ref + (i * stride) * D + d);
            const double v = (double)f;
            s += v;
            s2 += v * v;
            const uint32_t kk = key_of(f);
            kmn = max(kmn, ~kk);
            kmx = max(kmx, kk);
        }
    part[0][warp][lane] = s;
    part[1][warp][lane] = s2;
    pk[0][warp][lane] = kmn;
    pk[1][warp][lane] = kmx;
    __syncthreads();
    if (warp == 0 && d < D) {
        double t = 0.0, t2 = 0.0;
        uint32_t a = 0u, b = 0u;
        for (int w = 0; w < 8; ++w) {
            t += part[0][w][lane];
            t2 += part[1][w][lane];
            a = max(a, pk[0][w][lane]);
            b = max(b, pk[1][w][lane]);
        }
        atomicAdd(csum + d, t);
        atomicAdd(csum + Dp + d, t2);
        uint32_t* ck = reinterpret_cast<uint32_t*>(csum + 2 * Dp);
        atomicMax(ck + d, a);
        atomicMax(ck + Dp + d, b);
    }
}
__device__ __forceinline__ float knn_center_value(const double* csum, int64_t N, int D, int Dp, int d) {
    if (d >= D) return 0.f;
    const double ns = (double)(N < 16384 ? N : 16384);
    const double m = csum[d] / ns;
    const double var = csum[Dp + d] / ns - m * m;
    if (!(fabs(m) < 1e38) || !(var < 1e76)) return 0.f;  // non-finite sample: no centring
    if (var <= 0.0) return (float)m;
    const double gstep = ldexp(1.0, ilogb(sqrt(var)) - 4);
    return (float)(rint(m / gstep) * gstep);
}

// largest |x - c_d| over the sample in dim d (0 for padding dims; +Inf if not finite)
__device__ __forceinline__ float knn_sample_range(const double* csum, int D, int Dp, int d, float c) {
    if (d >= D) return 0.f;
    const uint32_t* ck = reinterpret_cast<const uint32_t*>(csum + 2 * Dp);
    const float vmin = __uint_as_float(bits_of_key(~ck[d])), vmax = __uint_as_float(bits_of_key(ck[Dp + d]));
    const double r = fmax((double)vmax - (double)c, (double)c - (double)vmin);
    return (r == r && r < 3.0e38) ? (float)r : __int_as_float(0x7f800000);
}

constexpr int KNN_PREP_THREADS = 256;

// knn_prep1_kernel: the operand images in ONE read of the points.  Every tile takes the
// call's common power-of-two scale sigma from the sample's range M (the largest |x - c|
// sampled): refs 2^(13 - ilogb M), queries 2^(12 - ilogb M), so a value up to 2 M still
// lands below 2^15 in fp16.  A tile holding a larger value (an outlier the sample missed)
// is listed for knn_stats_kernel + knn_prep_kernel, which rebuild it from its own max.
// Each block reads its tile 32 dims at a time (coalesced: a warp reads 32 consecutive
// floats of one row) into shared memory; thread i owns row i: |x'|^2 in double, the
// scaled fp16 chunks (16 B per thread, consecutive threads -> consecutive 16 B), then the
// bf16 norm block.  Rows past the end are all zeros.
__global__ void __launch_bounds__(256)
    knn_prep1_kernel(const float* __restrict__ ref, const float* __restrict__ qry, KnnGeom g, int nt,
                     const double* __restrict__ csum, float4* __restrict__ qstat, float2* __restrict__ tscale,
                     KnnStats* __restrict__ st, uint4* __restrict__ ref_img, uint4* __restrict__ q_img,
                     int* __restrict__ fixlist, int* __restrict__ fixcnt) {
    // (the shared transpose tile only on the scalar path: dynamic, 0 bytes when every row is
    // 16-byte aligned -- more blocks per SM for the direct 16-byte loads)
    extern __shared__ float prep_tile_raw[];
    auto tile = reinterpret_cast<float(*)[KNN_KS + 1]>(prep_tile_raw);
    __shared__ float cs[KNN_MAX_D];
    __shared__ uint32_t srange, smax;
    __shared__ int sover, sbad;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) { srange = 0u; smax = 0u; sover = 0; sbad = 0; }
    __syncthreads();
    for (int d = tid; d < g.Dp; d += 256) {
        const float c = knn_center_value(csum, g.N, g.D, g.Dp, d);
        cs[d] = c;
        const float r = knn_sample_range(csum, g.D, g.Dp, d, c);
        if (r > 0.f) atomicMax(&srange, __float_as_uint(r));
    }
    __syncthreads();
    const bool is_q = blockIdx.x >= (unsigned)nt;
    const int64_t t = is_q ? (int64_t)blockIdx.x - nt : (int64_t)blockIdx.x;
    const int rows = is_q ? KNN_BM : g.BN;
    const int64_t n = is_q ? g.Q : g.N;
    const float* x = is_q ? qry : ref;
    const int64_t row = t * rows + tid;
    const float M = __uint_as_float(srange);
    int e = 0;
    if (M > 0.f && M < 3.0e38f) e = min(max((is_q ? 12 : 13) - ilogbf(M), -120), 120);
    const float sig = ldexpf(1.f, e);
    const float mul = is_q ? -2.f * sig : sig;  // exact
    // (D % 4 == 0 and a 16-byte aligned base: every row is 16-byte aligned)
    const bool vec4 = (g.D & 3) == 0 && (reinterpret_cast<uintptr_t>(ref) & 15u) == 0 &&
                      (reinterpret_cast<uintptr_t>(qry) & 15u) == 0;  // (= the host's choice of smem)
    double s = 0.0;
    bool over = false, bad = false;
    for (int ks = 0; ks < g.KS; ++ks) {
        float vv[KNN_KS];  // this thread's row, dims ks * 32 .. + 31, centred
        if (vec4) {
            // (thread = row: its own 8 x 16-byte loads, L1-cached so that the other half of
            // each 32-byte sector serves the next load; no shared-memory transpose, no barriers)
            if (tid < rows) {
                const bool okr = row < n;
                const float4* xr = reinterpret_cast<const float4*>(x + (okr ? row : 0) * (int64_t)g.D + ks * KNN_KS);
                float4 v4[KNN_KS / 4];
#pragma unroll
                for (int u = 0; u < KNN_KS / 4; ++u)
                    v4[u] = (okr && ks * KNN_KS + 4 * u < g.D) ? __ldg(xr + u) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                for (int u = 0; u < KNN_KS / 4; ++u) {
                    const int d = ks * KNN_KS + 4 * u;
                    const bool ok = okr && d < g.D;
                    vv[4 * u + 0] = ok ? v4[u].x - cs[d] : 0.f;
                    vv[4 * u + 1] = ok ? v4[u].y - cs[d + 1] : 0.f;
                    vv[4 * u + 2] = ok ? v4[u].z - cs[d + 2] : 0.f;
                    vv[4 * u + 3] = ok ? v4[u].w - cs[d + 3] : 0.f;
                }
            }
        } else {
            __syncthreads();
            const int d = ks * KNN_KS + lane;
#pragma unroll 8
            for (int r = warp; r < rows; r += 8) {
                const int64_t gr = t * rows + r;
                tile[r][lane] = (gr < n && d < g.D) ? __ldcs(x + gr * (int64_t)g.D + d) - cs[d] : 0.f;
            }
            __syncthreads();
            if (tid < rows) {
#pragma unroll
                for (int j = 0; j < KNN_KS; ++j) vv[j] = tile[tid][j];
            }
        }
        if (tid < rows) {
            uint4* dst;
            int cstride;
            if (is_q) {  // [Dp/8 chunks][128 rows][8]
                dst = q_img + t * (int64_t)(g.a_bytes() / 16) + (int64_t)(ks * 4) * KNN_BM + tid;
                cstride = KNN_BM;
            } else {     // [stage][4 chunks][BN rows][8]
                dst = ref_img + t * (int64_t)(g.tile_bytes() / 16) + (int64_t)ks * (g.stage_bytes() / 16) + tid;
                cstride = g.BN;
            }
#pragma unroll
            for (int kc = 0; kc < 4; ++kc) {
                uint32_t h[4];
#pragma unroll
                for (int p = 0; p < 4; ++p) {
                    const float v0 = vv[kc * 8 + 2 * p], v1 = vv[kc * 8 + 2 * p + 1];
                    s += (double)v0 * (double)v0;
                    s += (double)v1 * (double)v1;
                    const float a0 = fabsf(v0), a1 = fabsf(v1);
                    bad |= !(a0 <= 3.4028235e38f) || !(a1 <= 3.4028235e38f);
                    over |= fabsf(mul * v0) >= 32768.f || fabsf(mul * v1) >= 32768.f;
                    h[p] = h2(mul * v0, mul * v1);
                }
                dst[kc * cstride] = make_uint4(h[0], h[1], h[2], h[3]);
            }
        }
    }
    if (tid < rows) {
        float sr = __double2float_ru(s);
        if (bad || !(sr == sr)) sr = __int_as_float(0x7f800000);
        if (row < n) {
            if (is_q) qstat[row] = make_float4(sig, 0.f, 0.f, sr);
            else atomicMax(&smax, __float_as_uint(sr));
        }
        const float n1 = __bfloat162float(__float2bfloat16_rn((float)s));
        const float n2 = __bfloat162float(__float2bfloat16_rn((float)(s - (double)n1)));
        const float n3 = __bfloat162float(__float2bfloat16_rn((float)(s - (double)n1 - (double)n2)));
        uint4* blk;
        uint4 c0;
        if (is_q) {
            blk = q_img + (t * (int64_t)g.a_bytes() + (int64_t)g.Dp * 256) / 16;
            c0 = make_uint4(bf2(sig * n1, sig * n2), bf2(sig * n3, sig), bf2(sig, sig), 0u);
        } else {
            blk = ref_img + (t * (int64_t)g.tile_bytes() + (int64_t)g.KS * g.stage_bytes()) / 16;
            c0 = make_uint4(bf2(sig, sig), bf2(sig, sig * n1), bf2(sig * n2, sig * n3), 0u);
        }
        if (row >= n) c0 = make_uint4(0u, 0u, 0u, 0u);
        blk[tid] = c0;
        blk[rows + tid] = make_uint4(0u, 0u, 0u, 0u);
        if (over && !bad) sover = 1;
        if (bad) sbad = 1;
    }
    __syncthreads();
    if (tid == 0) {
        if (sover && !sbad) fixlist[atomicAdd(fixcnt, 1)] = (int)blockIdx.x;  // rebuilt from its own max
        if (!is_q) {
            tscale[t] = make_float2(sig, 1.f / sig);  // (exact: a power of two)
            if (smax) atomicMax(&st->R2, smax);
            atomicMax(&st->isig, __float_as_uint(1.f / sig));
        }
    }
}

// knn_stats_kernel: one block per tile (blocks [0, nt): reference tiles of BN rows, then
// query tiles of 128 rows); a warp per row, coalesced.  Per row |x'|^2 in double (rownorm),
// per tile max |x'| -> sigma = 2^e with (2 for queries) x max |x'| x sigma in [2^14, 2^15)
// (tscale for reference tiles, qstat.x for queries), max |r'|^2 and max 1/sigma_t (st).
__global__ void __launch_bounds__(KNN_PREP_THREADS)
    knn_stats_kernel(const float* __restrict__ ref, const float* __restrict__ qry, KnnGeom g, int nt,
                     const double* __restrict__ csum, double* __restrict__ rownorm, float4* __restrict__ qstat,
                     float2* __restrict__ tscale, KnnStats* __restrict__ st, const int* __restrict__ list,
                     const int* __restrict__ lcnt) {
    __shared__ float cs[KNN_MAX_D];
    __shared__ uint32_t samx, smax;
    __shared__ int sbad;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int d = tid; d < g.Dp; d += KNN_PREP_THREADS) cs[d] = knn_center_value(csum, g.N, g.D, g.Dp, d);
    // (list != nullptr: the tiles knn_prep1_kernel listed, a grid-stride loop over them)
    const int nb = list ? *lcnt : (int)gridDim.x;
    for (int li = (int)blockIdx.x; li < nb; li += (int)gridDim.x) {
    const unsigned bid = list ? (unsigned)list[li] : blockIdx.x;
    __syncthreads();
    if (tid == 0) { samx = 0u; smax = 0u; sbad = 0; }
    __syncthreads();
    const bool is_q = bid >= (unsigned)nt;
    const int64_t t = is_q ? (int64_t)bid - nt : (int64_t)bid;
    const int rows = is_q ? KNN_BM : g.BN;
    const int64_t n = is_q ? g.Q : g.N;
    const float* x = is_q ? qry : ref;
    float mx = 0.f;
    bool bad = false;
    uint32_t rmax = 0u;
    for (int r0 = warp * 4; r0 < rows; r0 += 4 * (KNN_PREP_THREADS / 32)) {
        double s[4] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll 2
        for (int d0 = 0; d0 < g.D; d0 += 32) {
            const int d = d0 + lane;
            float v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t gr = t * rows + r0 + u;
                v[u] = (gr < n && d < g.D) ? __ldg(x + gr * (int64_t)g.D + d) - cs[d] : 0.f;
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                s[u] += (double)v[u] * (double)v[u];
                const float a = fabsf(v[u]);
                bad |= !(a <= 3.4028235e38f);
                mx = fmaxf(mx, a);
            }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) s[u] += __shfl_xor_sync(kFull, s[u], o);
            const int64_t gr = t * rows + r0 + u;
            if (lane == 0 && r0 + u < rows) {
                rownorm[bid * (int64_t)KNN_BN + r0 + u] = s[u];
                if (gr < n) {
                    float sr = __double2float_ru(s[u]);
                    if (!(sr == sr)) sr = __int_as_float(0x7f800000);
                    if (is_q) qstat[gr] = make_float4(0.f, 0.f, 0.f, sr);
                    else rmax = max(rmax, __float_as_uint(sr));
                }
            }
        }
    }
    mx = __uint_as_float(__reduce_max_sync(kFull, __float_as_uint(mx)));  // (non-negative: bits order)
    if (lane == 0) {
        if (mx > 0.f) atomicMax(&samx, __float_as_uint(mx));
        if (rmax) atomicMax(&smax, rmax);
    }
    if (__any_sync(kFull, bad) && lane == 0) sbad = 1;
    __syncthreads();
    const float tmx = __uint_as_float(samx);
    int e = 0;
    if (!sbad && tmx > 0.f) e = min(max((is_q ? 13 : 14) - ilogbf(tmx), -120), 120);
    const float sig = ldexpf(1.f, e);
    if (is_q) {
        for (int r = tid; r < rows; r += KNN_PREP_THREADS) {
            const int64_t gr = t * rows + r;
            if (gr < n) {
                qstat[gr].x = sig;
                if (sbad) qstat[gr].w = __int_as_float(0x7f800000);
            }
        }
    } else if (tid == 0) {
        tscale[t] = make_float2(sig, 1.f / sig);  // (exact: a power of two)
        atomicMax(&st->R2, sbad ? 0x7f800000u : smax);
        atomicMax(&st->isig, __float_as_uint(1.f / sig));
    }
    }
}

// knn_prep_kernel: the operand images.  Each block reads its tile 32 dims at a time
// (coalesced: a warp reads 32 consecutive floats of one row) into shared memory; thread i
// then owns row i and writes its scaled fp16 chunks (16 B per thread, consecutive threads ->
// consecutive 16 B).  Last, the bf16 norm block (the extra 16-wide K block): |x'|^2 split
// three ways (n1 + n2 + n3 to ~2^-24), queries [s n1, s n2, s n3, s, s, s, 0, 0],
// references [s, s, s, s m1, s m2, s m3, 0, 0] (s the tile's sigma; products of powers of
// two are exact), so the accumulator is sigma_q sigma_t (|q'|^2 + |r'|^2 - 2 q'.r').
// Rows past the end are all zeros.
__global__ void __launch_bounds__(KNN_PREP_THREADS)
    knn_prep_kernel(const float* __restrict__ ref, const float* __restrict__ qry, KnnGeom g, int nt,
                    const double* __restrict__ csum, const double* __restrict__ rownorm,
                    const float4* __restrict__ qstat, const float2* __restrict__ tscale,
                    uint4* __restrict__ ref_img, uint4* __restrict__ q_img, const int* __restrict__ list,
                    const int* __restrict__ lcnt) {
    __shared__ float tile[KNN_BN][KNN_KS + 1];
    __shared__ float cs[KNN_MAX_D];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int d = tid; d < g.Dp; d += KNN_PREP_THREADS) cs[d] = knn_center_value(csum, g.N, g.D, g.Dp, d);
    const int nb = list ? *lcnt : (int)gridDim.x;
    for (int li = (int)blockIdx.x; li < nb; li += (int)gridDim.x) {
    const unsigned bid = list ? (unsigned)list[li] : blockIdx.x;
    const bool is_q = bid >= (unsigned)nt;
    const int64_t t = is_q ? (int64_t)bid - nt : (int64_t)bid;
    const int rows = is_q ? KNN_BM : g.BN;
    const int64_t n = is_q ? g.Q : g.N;
    const float* x = is_q ? qry : ref;
    const int64_t row = t * rows + tid;
    const float sig = is_q ? (t * rows < n ? qstat[t * rows].x : 1.f) : tscale[t].x;
    const float mul = is_q ? -2.f * sig : sig;  // exact
    for (int ks = 0; ks < g.KS; ++ks) {
        __syncthreads();
        const int d = ks * KNN_KS + lane;
#pragma unroll 8
        for (int r = warp; r < rows; r += KNN_PREP_THREADS / 32) {
            const int64_t gr = t * rows + r;
            tile[r][lane] = (gr < n && d < g.D) ? __ldcs(x + gr * (int64_t)g.D + d) - cs[d] : 0.f;
        }
        __syncthreads();
        if (tid < rows) {
            uint4* dst;
            int cstride;
            if (is_q) {  // [Dp/8 chunks][128 rows][8]
                dst = q_img + t * (int64_t)(g.a_bytes() / 16) + (int64_t)(ks * 4) * KNN_BM + tid;
                cstride = KNN_BM;
            } else {     // [stage][4 chunks][BN rows][8]
                dst = ref_img + t * (int64_t)(g.tile_bytes() / 16) + (int64_t)ks * (g.stage_bytes() / 16) + tid;
                cstride = g.BN;
            }
#pragma unroll
            for (int kc = 0; kc < 4; ++kc) {
                uint32_t h[4];
#pragma unroll
                for (int p = 0; p < 4; ++p) h[p] = h2(mul * tile[tid][kc * 8 + 2 * p], mul * tile[tid][kc * 8 + 2 * p + 1]);
                dst[kc * cstride] = make_uint4(h[0], h[1], h[2], h[3]);
            }
        }
    }
    if (tid < rows) {
        const double s = rownorm[bid * (int64_t)KNN_BN + tid];
        const float n1 = __bfloat162float(__float2bfloat16_rn((float)s));
        const float n2 = __bfloat162float(__float2bfloat16_rn((float)(s - (double)n1)));
        const float n3 = __bfloat162float(__float2bfloat16_rn((float)(s - (double)n1 - (double)n2)));
        uint4* blk;
        uint4 c0;
        if (is_q) {
            blk = q_img + (t * (int64_t)g.a_bytes() + (int64_t)g.Dp * 256) / 16;
            c0 = make_uint4(bf2(sig * n1, sig * n2), bf2(sig * n3, sig), bf2(sig, sig), 0u);
        } else {
            blk = ref_img + (t * (int64_t)g.tile_bytes() + (int64_t)g.KS * g.stage_bytes()) / 16;
            c0 = make_uint4(bf2(sig, sig), bf2(sig, sig * n1), bf2(sig * n2, sig * n3), 0u);
        }
        if (row >= n) c0 = make_uint4(0u, 0u, 0u, 0u);
        blk[tid] = c0;
        blk[rows + tid] = make_uint4(0u, 0u, 0u, 0u);
    }
    __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// tcgen05 helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    // K-major, SWIZZLE_NONE canonical layout; version 1 (bits 46-47), base offset 0
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}

// kind::f16 instruction descriptor: bf16 x bf16 -> fp32, K-major A and B, M x N (the norm block)
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int M, int N) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// kind::f16 instruction descriptor: fp16 x fp16 -> fp32 (a/b format 0), K-major, M x N
__host__ __device__ constexpr uint32_t umma_idesc_f16(int M, int N) {
    return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// one tcgen05.mma kind::f16 (fp16 or bf16 operands, per the instruction descriptor)
__device__ __forceinline__ void umma_bf16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
}

__device__ __forceinline__ void umma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                     smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void tmem_ld64(uint32_t taddr, uint32_t (&v)[64]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x64.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31, %32, %33, %34, %35, %36, %37, %38, %39, %40, %41, %42, %43, %44, %45, %46, %47, %48, %49, %50, %51, %52, %53, %54, %55, %56, %57, %58, %59, %60, %61, %62, %63}, [%64];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31]), "=r"(v[32]), "=r"(v[33]), "=r"(v[34]), "=r"(v[35]), "=r"(v[36]), "=r"(v[37]), "=r"(v[38]), "=r"(v[39]), "=r"(v[40]), "=r"(v[41]), "=r"(v[42]), "=r"(v[43]), "=r"(v[44]), "=r"(v[45]), "=r"(v[46]), "=r"(v[47]), "=r"(v[48]), "=r"(v[49]), "=r"(v[50]), "=r"(v[51]), "=r"(v[52]), "=r"(v[53]), "=r"(v[54]), "=r"(v[55]), "=r"(v[56]), "=r"(v[57]), "=r"(v[58]), "=r"(v[59]), "=r"(v[60]), "=r"(v[61]), "=r"(v[62]), "=r"(v[63])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// Split form of tmem_ld32: issue without waiting, and a wait that names the
// destination registers (so no use of them can be scheduled above it).  Lets
// the epilogue process one 32-column chunk while the next one is in flight.
__device__ __forceinline__ void tmem_ld32_issue(uint32_t taddr, uint32_t (&v)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait32(uint32_t (&v)[32]) {
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(v[0]), "+r"(v[1]), "+r"(v[2]), "+r"(v[3]), "+r"(v[4]), "+r"(v[5]), "+r"(v[6]), "+r"(v[7]),
                   "+r"(v[8]), "+r"(v[9]), "+r"(v[10]), "+r"(v[11]), "+r"(v[12]), "+r"(v[13]), "+r"(v[14]),
                   "+r"(v[15]), "+r"(v[16]), "+r"(v[17]), "+r"(v[18]), "+r"(v[19]), "+r"(v[20]), "+r"(v[21]),
                   "+r"(v[22]), "+r"(v[23]), "+r"(v[24]), "+r"(v[25]), "+r"(v[26]), "+r"(v[27]), "+r"(v[28]),
                   "+r"(v[29]), "+r"(v[30]), "+r"(v[31])
                 :
                 : "memory");
}

__device__ __forceinline__ uint32_t ld_vol_shared_u32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_vol_shared_u64(uint32_t a) {
    unsigned long long v;
    asm volatile("ld.volatile.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void st_shared_u32(uint32_t a, uint32_t v) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void st_shared_u64(uint32_t a, unsigned long long v) {
    asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ void atom_min_shared_u64(uint32_t a, unsigned long long v) {
    asm volatile("red.shared.min.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t atom_add_shared(uint32_t saddr, uint32_t v) {
    uint32_t r;
    asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(r) : "r"(saddr), "r"(v) : "memory");
    return r;
}

// min of three floats in one instruction (sm_100: FMNMX3; a NaN operand is ignored like fminf)
__device__ __forceinline__ float fmin3(float a, float b, float c) {
    float r;
    asm("min.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
    return r;
}

__device__ __forceinline__ void red_add_shared(uint32_t saddr, uint32_t v) {
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
}

// cluster helpers (reference-stage multicast across the CTAs of a cluster)
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// 1-D bulk copy global -> the same shared-memory offset in every CTA of `mask`;
// each destination CTA's mbarrier at `bar`'s offset receives the complete_tx bytes
__device__ __forceinline__ void bulk_g2s_mc(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint16_t mask) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], "
        "%4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "h"(mask)
        : "memory");
}
// MMA completion -> arrive on the mbarrier at `bar`'s offset in every CTA of `mask`
__device__ __forceinline__ void umma_commit_mc(uint64_t* bar, uint16_t mask) {
    asm volatile(
        "tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
            smem_u32(bar)),
        "h"(mask)
        : "memory");
}

// ---------------------------------------------------------------------------
// the fused kernel
// ---------------------------------------------------------------------------
struct KnnSmem {
    static constexpr int kHistWarp = 256 * 4;                  // per epilogue warp: radix histogram (pool_select64)
    static constexpr int kWarpScratch = KNN_SB * 32 * 4;      // per query group of 32: sampling histogram, one per lane
    // scratch of `ew` epilogue warps (sized for the launch: every KB left goes to the ring)
    // EW warps' radix histograms, one sampling histogram per query group (a TMEM lane
    // quadrant of a query tile: the EW / 4 warps scanning its column parts share it), and
    // the per-query state those warps share: pool fill, failure flag, bound pair
    __host__ __device__ static int scratch(int ew, int qpc) {
        return ew * kHistWarp + 4 * qpc * kWarpScratch + qpc * 128 * 24;
    }
    __host__ __device__ static int total(const KnnGeom& g) {
        return 1024 /*align slack*/ + g.QPC * g.a_bytes() + g.NS * g.stage_bytes() + scratch(g.EW, g.QPC) +
               (2 * g.NS + 5) * 8 + 16;
    }
};

// MODE 0: selection (knn_search); 1: write every distance (knn_distances);
// 2: pipeline only -- the epilogue reads the accumulators and drops them
// (experiments: isolates the TMA + MMA + TMEM pipeline from the selection);
// 3: selection + per-warp cycle counters; 4: pipeline without any TMEM read.
// BN: references per tile; QPC: query tiles per CTA (each B stage feeds QPC x 128
// queries: with QPC = 2, BN = 128 and four 128-column accumulators, half the bytes
// land in shared memory per output)
template <int MODE, int EW, int BN, int QPC>
__global__ void __launch_bounds__(knn_threads(EW), 1)  // (EW = 16: 18 warps, 5 on one SM sub-partition -> <= 96 registers)
    knn_fused_kernel(KnnGeom g, const uint8_t* __restrict__ ref_img, const uint8_t* __restrict__ q_img,
                     const float4* __restrict__ qstat, const KnnStats* __restrict__ st,
                     unsigned long long* __restrict__ pool64, int32_t* __restrict__ cnt_out,
                     unsigned long long* __restrict__ qthr, int32_t* __restrict__ qfail, float* __restrict__ dump,
                     const unsigned long long* __restrict__ qspec, const float2* __restrict__ tscale) {
    constexpr int HALVES = (QPC == 1) ? EW / 4 : 1;
    constexpr int WCOLS = BN / HALVES;  // columns of each tile this epilogue warp scans
    constexpr int SB = KNN_KS * BN * 2;       // bytes of one reference stage (fp16)
    constexpr int NBB = 16 * BN * 2;          // bytes of a reference tile's norm block
    constexpr bool DUMP = (MODE == 1);
    constexpr bool PIPE_ONLY = (MODE == 2 || MODE == 4);
    constexpr bool NO_READ = (MODE == 4);  // pipeline only, accumulators never read (experiments)
    constexpr bool PROF = (MODE == 3);  // selection + per-warp cycle counters (experiments)
    unsigned long long prof_app = 0, prof_narrow = 0, prof_wait = 0, prof_chunks = 0, prof_rare = 0, prof_nrare = 0, prof_nnarrow = 0;
    const unsigned long long prof_t0 = PROF ? clock64() : 0;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
    const int NS = g.NS;
    uint8_t* sA = smem;
    uint8_t* sB = sA + QPC * g.a_bytes();
    uint32_t* hist_all = reinterpret_cast<uint32_t*>(sB + NS * SB);
    float* dstage_all = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(hist_all) + EW * KnnSmem::kHistWarp);
    unsigned long long* qs_T = reinterpret_cast<unsigned long long*>(reinterpret_cast<uint8_t*>(dstage_all) +
                                                                     4 * QPC * KnnSmem::kWarpScratch);  // [QPC*128]
    int* qs_n = reinterpret_cast<int*>(qs_T + QPC * 128);                                              // [QPC*128]
    int* qs_f = qs_n + QPC * 128;                                                                      // [QPC*128]
    uint32_t* qs_v = reinterpret_cast<uint32_t*>(qs_f + QPC * 128);                                   // [QPC*128]
    uint64_t* bars = reinterpret_cast<uint64_t*>(qs_v + QPC * 256);
    uint64_t* full = bars;
    uint64_t* empty = bars + NS;
    uint64_t* accf = bars + 2 * NS;
    uint64_t* acce = accf + 2;
    uint64_t* afull = acce + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(afull + 1);

    const int warp = threadIdx.x >> 5;
    const uint32_t lane = lane_id();
    const int grp = blockIdx.x % g.QTp;  // query tiles grp*QPC.. (>= QT: padding, no queries)
    const int split = blockIdx.x / g.QTp;
    const uint32_t crank = g.cs > 1 ? cluster_rank() : 0u;
    const uint16_t cmask = (uint16_t)((1u << g.cs) - 1u);
    const int t0 = g.split_begin(split);  // logical tile range of this CTA
    const int t1 = g.split_begin(split + 1);
    // Cold CTAs (the first wave: no split of their queries has published a bound
    // yet) first stream their first Fs tiles through the pipeline for a distance
    // histogram per query (starting bound, see the epilogue), then all t1 - t0.
    const int Fs = (!DUMP && !PIPE_ONLY && qspec == nullptr && (int)blockIdx.x < g.sample_ctas && g.k <= BN && g.tstride == 1 &&
                    t1 - t0 >= 4 * g.sample_tiles && (int64_t)(t0 + g.sample_tiles) * BN <= g.N)
                       ? g.sample_tiles
                       : 0;
    const int nsteps = Fs + (t1 - t0);

    if (warp == 0 && lane == 0) {
        for (int s = 0; s < NS; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], g.cs);  // every CTA of the cluster must have consumed the stage
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&accf[b], 1);
            mbar_init(&acce[b], EW);
        }
        mbar_init(afull, 1);
        fence_mbar_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(512)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    if (g.cs > 1) cluster_sync_all();  // peers' barriers initialised before any multicast
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        // ===== producer: resident query tile, then the reference stream =====
        // (per tile: KS dims stages of 32 KB, then the 8 KB norm block)
        if (lane == 0) {
            const uint32_t abytes = (uint32_t)g.a_bytes();
            mbar_arrive_expect_tx(afull, QPC * abytes);
#pragma unroll
            for (int h = 0; h < QPC; ++h) {
                const int qtile = grp * QPC + h;
                bulk_g2s(sA + h * abytes, q_img + (size_t)(qtile < g.QT ? qtile : 0) * abytes, abytes, afull);
            }
            uint32_t it = 0;
            for (int lt = 0; lt < nsteps; ++lt) {
                const int t = (lt < Fs ? t0 + lt : t0 + lt - Fs) * g.tstride;
                for (int ks = 0; ks <= g.KS; ++ks, ++it) {
                    const int st = (int)(it % NS);
                    const uint32_t bytes = (ks < g.KS) ? SB : NBB;
                    mbar_wait_sleep(&empty[st], ((it / NS) & 1u) ^ 1u);
                    mbar_arrive_expect_tx(&full[st], bytes);
                    const uint8_t* src = ref_img + (size_t)t * g.tile_bytes() + (size_t)ks * SB;
                    if (g.cs == 1) {
                        bulk_g2s(sB + st * SB, src, bytes, &full[st]);
                    } else {  // this CTA's slice of the stage, into every CTA of the cluster
                        const uint32_t sl = bytes / g.cs;
                        bulk_g2s_mc(sB + st * SB + crank * sl, src + crank * sl, sl, &full[st], cmask);
                    }
                }
            }
        }
    } else if (warp == 1) {
        // ===== MMA issuer (one thread) =====
        if (lane == 0) {
            constexpr uint32_t idesc = umma_idesc_f16(KNN_BM, BN);      // fp16 x fp16 -> fp32
            constexpr uint32_t idesc_n = umma_idesc_bf16(KNN_BM, BN);   // the bf16 norm block
            const uint32_t abytes = (uint32_t)g.a_bytes();
            mbar_wait(afull, 0);
            tc_fence_after();
            uint32_t it = 0;
            for (int lt = 0; lt < nsteps; ++lt) {
                const int b = lt & 1;
                mbar_wait_sleep(&acce[b], (((uint32_t)lt >> 1) & 1u) ^ 1u);
                tc_fence_after();
                for (int ks = 0; ks <= g.KS; ++ks, ++it) {
                    const int st = (int)(it % NS);
                    mbar_wait_sleep(&full[st], (it / NS) & 1u);
                    tc_fence_after();
                    const uint32_t bs = smem_u32(sB + st * SB);
#pragma unroll
                    for (int h = 0; h < QPC; ++h) {  // every query tile of the CTA on this stage
                        const uint32_t d_tmem = tmem_base + (uint32_t)((b * QPC + h) * BN);
                        const uint32_t a0 = smem_u32(sA) + (uint32_t)h * abytes;
                        if (ks == g.KS) {  // norm block: |q'|^2 + |r'|^2 into the same accumulator
                            const uint64_t an = umma_desc(a0 + (uint32_t)(g.Dp * 256), KNN_BM * 16, 128);
                            const uint64_t bn = umma_desc(bs, BN * 16, 128);
                            umma_bf16(d_tmem, an, bn, idesc_n, 1u);
                            continue;
                        }
#pragma unroll
                        for (int j = 0; j < 2; ++j) {
                            const int kk = ks * 2 + j;
                            const uint64_t ad = umma_desc(a0 + (uint32_t)(2 * kk) * (KNN_BM * 16), KNN_BM * 16, 128);
                            const uint64_t bd = umma_desc(bs + (uint32_t)(2 * j) * (BN * 16), BN * 16, 128);
                            umma_bf16(d_tmem, ad, bd, idesc, (ks | j) ? 1u : 0u);
                        }
                    }
                    // frees the stage (in every CTA of the cluster) when these MMAs complete
                    if (g.cs == 1) umma_commit(&empty[st]);
                    else umma_commit_mc(&empty[st], cmask);
                }
                umma_commit(&accf[b]);  // accumulator b ready for the epilogue
            }
        }
    } else {
        // ===== epilogue: one thread per query =====
        const int e = warp - 2;                   // 0..EW-1
        const int quad = warp & 3;                // TMEM lane quadrant this warp may access
        const int half = (QPC == 1) ? (e >> 2) : 0;  // columns [half * WCOLS, (half + 1) * WCOLS) of every tile
        const int hq = (QPC == 1) ? 0 : (e >> 2);    // query tile of the CTA this warp serves
        const int qt = grp * QPC + hq;
        const int row = quad * 32 + (int)lane;    // query row within the tile
        const int64_t q = (int64_t)qt * KNN_BM + row;
        const bool qvalid = q < g.Q;
        uint32_t* hist = hist_all + e * 256;
        // The PAIR = EW / 4 warps on one query group (same TMEM lanes, different column
        // parts) share the query's pool, its fill counter and its bound (shared memory);
        // they meet at a named barrier before and after every narrowing phase.
        constexpr int PAIR = HALVES;
        const int qgrp = hq * 4 + quad;
        const int qidx = hq * 128 + row;
        uint8_t* wscratch = reinterpret_cast<uint8_t*>(dstage_all) + qgrp * KnnSmem::kWarpScratch;
        // the query group's shared state, by 32-bit shared-space address (explicit
        // ld/st/atom.shared: no generic volatile accesses, fewer live registers)
        const uint32_t np_s = smem_u32(qs_n + qidx);   // pool fill
        const uint32_t fp_s = smem_u32(qs_f + qidx);   // failure flag
        const uint32_t Tp_s = smem_u32(qs_T + qidx);   // shared bound pair
        auto pair_bar = [&]() {
            if constexpr (PAIR > 1) asm volatile("bar.sync %0, %1;" ::"r"(1 + qgrp), "r"(32 * PAIR) : "memory");
            else __syncwarp();
        };
        // this query's candidate pool: packed pairs (key << 32 | reference row), one per split
        const size_t list = (size_t)split;
        unsigned long long* pool = pool64 + (list * g.Q + (qvalid ? q : 0)) * g.P;
        unsigned long long T = kSentPair;  // running bound on the k-th (d~, index) pair
        // the band: 2 eps_q above the k-th d~ (every reference that can be in the exact top-k)
        const float band = (qvalid && !DUMP) ? __fmul_ru(2.f, knn_eps(qstat[q], *st, g.D)) : 0.f;
        const float sq = qvalid ? qstat[q].x : 1.f;  // sigma of this query tile
        const float sqi = __frcp_rn(sq);               // (exact: a power of two)
        float tv = 0.f;                    // filter value: value(T) + band, rounded up
        bool fast = false;                 // finite filter value: the fp32 compare d~ <= tv pre-filters
        bool failed = !(band < __int_as_float(0x7f800000));  // no finite band: exact fallback
        if (qvalid && !DUMP && !PIPE_ONLY && failed && half == 0 && !g.prepass) qfail[q] = 1;
        if (half == 0) {
            st_shared_u32(np_s, 0u);
            st_shared_u32(fp_s, failed ? 1u : 0u);
            st_shared_u64(Tp_s, kSentPair);
        }
        pair_bar();

        auto set_T = [&](unsigned long long t) {
            T = t;
            const uint32_t tk = (uint32_t)(T >> 32);
            tv = (tk < 0xff800000u) ? __fadd_ru(__uint_as_float(bits_of_key(tk)), band) : 0.f;
            fast = tk < 0xff800000u && tv < __int_as_float(0x7f800000);
        };
        auto adopt = [&](unsigned long long t) {
            if (t < T) {
                set_T(t);
                if (PAIR > 1) atom_min_shared_u64(Tp_s, t);
            }
        };
        // Speculative start (knn_run's sampled pre-pass): T_spec, the j-th smallest d~ of a
        // strided sample, is very likely above the row's k-th d~ -- admitting against it from
        // the first tile replaces the slow convergence of S independent running bounds.
        // Unverified here: knn_rescore_kernel checks that >= k pooled pairs are <= T_spec
        // (else the query takes the exact fallback).
        if (qspec != nullptr && qvalid && !DUMP && !PIPE_ONLY) {
            const unsigned long long ts = __ldg(qspec + q);
            if ((uint32_t)(ts >> 32) != kSentKey) set_T(ts);
        }
        // after a pair barrier: the pair's shared bound and failure flag
        auto refresh = [&]() {
            if constexpr (PAIR > 1) {
                const unsigned long long t = ld_vol_shared_u64(Tp_s);
                if (t < T) set_T(t);
                failed = ld_vol_shared_u32(fp_s) != 0u;
            }
        };
        // warp-cooperative narrowing of every lane whose pool cannot take `room` more pairs:
        // the exact k-th pair of the pool becomes the bound and the pool keeps the band
        // above it; mid-stream, a band that alone leaves no room fails the query
        // (the PAIR warps of a query group split the narrowings of its lanes between them)
        auto narrow_lanes = [&](int room, int target, int cap, bool final_pass) {
            pair_bar();
            refresh();
            const int n = (int)ld_vol_shared_u32(np_s);
            // both warps of the pair have read the shared fills and bounds before either
            // narrows (and writes them): they derive the same `need` and split it consistently
            pair_bar();
            uint32_t need = __ballot_sync(kFull, qvalid && !failed && n + room > cap && n > target);
            // mid-stream, any bound with k..k + slack pairs at or below it will do (the
            // exact k-th is only needed by the final pass): the narrowing stops early
            const uint32_t slk = final_pass ? 0u : (uint32_t)max(0, (cap - target - room) / 4);
            int turn = 0;
            while (need) {
                if (PROF) prof_nnarrow++;
                const int j = __ffs(need) - 1;
                need &= need - 1u;
                if ((turn++ % PAIR) != half) continue;
                unsigned long long* jp = (unsigned long long*)__shfl_sync(kFull, (unsigned long long)pool, j);
                const int jn = __shfl_sync(kFull, n, j);
                const float jb = __shfl_sync(kFull, band, j);
                int nn;
                const unsigned long long t =
                    (jn <= 256)   ? pool_narrow64<8>(jp, jn, (uint32_t)target, &nn, jb, slk)
                    : (jn <= 512) ? pool_narrow64<16>(jp, jn, (uint32_t)target, &nn, jb, slk)
                    : (EW <= 8 && jn <= 32 * kNarrowRegs) ? pool_narrow64<(EW <= 8 ? kNarrowRegs : 16)>(jp, jn, (uint32_t)target, &nn, jb, slk)
                                               : pool_select64(jp, jn, (uint32_t)target, hist, &nn, jb, slk);
                if ((int)lane == j) {
                    st_shared_u32(np_s, (uint32_t)nn);
                    adopt(t);
                    // publish: the k-th pair of this split's part bounds the whole row
                    if (target == g.k && (uint32_t)(t >> 32) != kSentKey) atomicMin(&qthr[q], t);
                    if (!final_pass && nn + room > cap) {  // the band alone fills the pool
                        failed = true;
                        st_shared_u32(np_s, 0u);
                        st_shared_u32(fp_s, 1u);
                        if (!g.prepass) qfail[q] = 1;  // (pre-pass: just no speculation)
                    }
                }
            }
            __syncwarp();
            pair_bar();
            refresh();
        };

        // sample histogram of this lane's query: 64 buckets [lo, hi) in the warp scratch
        uint32_t* shist = reinterpret_cast<uint32_t*>(wscratch) + lane;
        const uint32_t shist_s = smem_u32(shist);
        float s_lo = 0.f, s_hi = -1.f, s_inv = 0.f;
        unsigned long long thr_next = (qvalid && !DUMP && !PIPE_ONLY) ? __ldcg(&qthr[q]) : kSentPair;
        int ncheck = 1;  // tiles until the next bound refresh / narrowing check
        for (int lt = 0; lt < nsteps; ++lt) {
            const bool sampling = lt < Fs;
            const int t = (sampling ? t0 + lt : t0 + lt - Fs) * g.tstride;
            const int b = lt & 1;
            if (!DUMP && !PIPE_ONLY && --ncheck <= 0) {
                ncheck = g.nstride;
                // adopt the tightest bound any split of this query had published when the
                // previous check started (the load's latency hides behind those tiles)
                adopt(thr_next);
                if (qvalid) thr_next = __ldcg(&qthr[q]);
                const unsigned long long c0 = PROF ? clock64() : 0;
                narrow_lanes(g.nstride * BN, g.k, g.pcap, false);  // room: every column of nstride tiles
                if (PROF) prof_narrow += clock64() - c0;
            }
            const unsigned long long cw0 = PROF ? clock64() : 0;
            mbar_wait(&accf[b], ((uint32_t)lt >> 1) & 1u);
            if (PROF) prof_wait += clock64() - cw0;
            const unsigned long long cc0 = PROF ? clock64() : 0;
            tc_fence_after();
            const uint32_t taddr = tmem_base + ((uint32_t)(quad * 32) << 16) + (uint32_t)((b * QPC + hq) * BN);
            // the accumulator is sigma_q sigma_t d~: compare it with the bound scaled the same
            // way (rounded up: never rejects a candidate) and unscale what is kept (powers of
            // two: exact unless subnormal, covered by knn_eps)
            const float2 tsc = __ldg(tscale + t);  // (sigma_t, 1 / sigma_t)
            const float stl = sq * tsc.x;
            const float inv = sqi * tsc.y;
            if (!DUMP && !PIPE_ONLY && lt == 0 && g.k <= BN && (int64_t)t * BN + BN <= g.N && qspec == nullptr) {
                // Starting bound without a fill phase: the exact k-th smallest distance of
                // this first (full) tile, by bisection on the bits of the clamped value
                // (non-negative floats order like their bit patterns), re-reading the
                // accumulator from TMEM each step.  At least k pairs of the row are <= it,
                // so (that key, any index) is a valid bound.
                // (one warp of the query group bisects; the others read its result)
                uint32_t vb = 0;
#pragma unroll 1
                for (int bit = 30; bit >= 0 && half == 0; --bit) {
                    const uint32_t cand = vb | (1u << bit);
                    uint32_t cnt = 0;
#pragma unroll 1
                    for (int c = 0; c < BN / 32; ++c) {
                        uint32_t v[32];
                        tmem_ld32(taddr + (uint32_t)(c * 32), v);
#pragma unroll
                        for (int j = 0; j < 32; ++j) {
                            const float x = __uint_as_float(v[j]) * inv;
                            cnt += (__float_as_uint(x < 0.f ? 0.f : x) < cand) ? 1u : 0u;
                        }
                    }
                    if (cnt < (uint32_t)g.k) vb = cand;
                }
                if (half == 0) {
                    qs_v[qidx] = vb;
                    if (qvalid) adopt(((unsigned long long)key_of(__uint_as_float(vb)) << 32) | 0x7ffffffeu);
                }
                pair_bar();
                vb = qs_v[qidx];
                refresh();
                if (Fs > 0) {
                    // histogram range: [max(0, tile minimum), k-th of the tile]
                    float mn = __int_as_float(0x7f800000);
#pragma unroll 1
                    for (int c = 0; c < BN / KNN_CW; ++c) {
                        uint32_t v[KNN_CW];
                        tmem_ld64(taddr + (uint32_t)(c * KNN_CW), v);
#pragma unroll
                        for (int j = 0; j < KNN_CW; ++j) mn = fminf(mn, __uint_as_float(v[j]) * inv);
                    }
                    s_lo = fmaxf(mn, 0.f);
                    s_hi = __uint_as_float(vb);
                    // buckets must stay far wider than an ulp (the bound below keeps one
                    // spare bucket for rounding); otherwise no histogram for this query
                    if (!(s_hi < __int_as_float(0x7f800000)) || !(s_hi - s_lo > s_hi * 0x1p-10f)) s_hi = -1.f;
                    s_inv = (s_hi > 0.f) ? (float)KNN_SB / (s_hi - s_lo) : 0.f;
                    if (half == 0) {
#pragma unroll 8
                        for (int j = 0; j < KNN_SB; ++j) shist[j * 32] = 0u;
                    }
                    pair_bar();  // the shared histogram is clear before either warp counts
                }
            }
            if (sampling) {
                // count this warp's half-tile distances <= hi per bucket (NaN fails the test)
#pragma unroll 1
                for (int c = half * (WCOLS / KNN_CW); c < (half + 1) * (WCOLS / KNN_CW); ++c) {
                    uint32_t v[KNN_CW];
                    tmem_ld64(taddr + (uint32_t)(c * KNN_CW), v);
#pragma unroll
                    for (int j = 0; j < KNN_CW; ++j) {
                        const float d = __uint_as_float(v[j]) * inv;
                        if (d <= s_hi) {
                            const int bk = min(max((int)((d - s_lo) * s_inv), 0), KNN_SB - 1);
                            red_add_shared(shist_s + (uint32_t)(bk * 128), 1u);
                        }
                    }
                }
                if (lt == Fs - 1) pair_bar();  // both column parts counted
                if (lt == Fs - 1 && qvalid && s_hi > 0.f && half == 0) {
                    // >= k of the sampled distances lie in buckets <= j, i.e. below lo + (j + 1) w;
                    // one spare bucket absorbs the rounding of the bucket index
                    uint32_t cum = 0;
                    int j = 0;
                    for (; j < KNN_SB; ++j) {
                        cum += shist[j * 32];
                        if (cum >= (uint32_t)g.k) break;
                    }
                    if (j < KNN_SB - 2) {
                        const float bound = s_lo + (float)(j + 2) * ((s_hi - s_lo) * (1.f / KNN_SB));
                        const unsigned long long tb = ((unsigned long long)key_of(bound) << 32) | 0x7ffffffeu;
                        adopt(tb);
                        atomicMin(&qthr[q], tb);
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive_cta(&acce[b]);
                continue;
            }
            if constexpr (!DUMP && !PIPE_ONLY) {
                // Selection scan of the tile: 32 columns per TMEM load, the next load in
                // flight while the current chunk is filtered.  Per chunk: min of each
                // 4-column group, one warp vote of the chunk minimum against each lane's
                // bound; on a hit, one warp-uniform vote per group, and only groups some
                // lane needs are visited (candidates appended, predicated, from registers).
                const uint32_t colt = (uint32_t)t * BN;  // N < 2^31
                const int nlim = (int)min((int64_t)BN, g.N - (int64_t)colt);  // valid columns of the tile
                const bool live = qvalid && !failed;
                // the filter value of this tile in accumulator units: value(T) + band scaled up
                // (rounded up: never rejects a candidate), +Inf without a finite bound (all
                // values pass), NaN for a lane that takes nothing (every compare fails)
                const float tvl = !live ? __int_as_float(0x7fc00000)
                                        : (fast ? __fmul_ru(tv, stl) : __int_as_float(0x7f800000));
                auto scan32 = [&](const uint32_t(&v)[32], int c0) {
                    float gmn[8];  // 3-input minima (FMNMX3): 20 instructions per 32 values
#pragma unroll
                    for (int j = 0; j < 8; ++j)
                        gmn[j] = fminf(fmin3(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]),
                                             __uint_as_float(v[4 * j + 2])),
                                       __uint_as_float(v[4 * j + 3]));
                    const float mn = fmin3(fmin3(gmn[0], gmn[1], gmn[2]), fmin3(gmn[3], gmn[4], gmn[5]),
                                           fminf(gmn[6], gmn[7]));
                    if (!__any_sync(kFull, mn <= tvl)) return;
                    const unsigned long long cr0 = PROF ? clock64() : 0;
                    // rare path: each lane visits only its own candidate groups (a divergent
                    // loop of max-over-lanes length); the group's 4 values are picked from the
                    // registers by a 3-level select tree (registers cannot be indexed
                    // dynamically; measured faster than a warp vote per group with static
                    // indices).  An element with d == tv and a larger index than T's is a
                    // harmless extra pool entry (narrowing applies the exact pair order).
                    uint32_t gm = 0;
#pragma unroll
                    for (int u = 0; u < 8; ++u) gm |= (uint32_t)(gmn[u] <= tvl) << u;
                    while (gm) {
                        const int u = __ffs(gm) - 1;
                        gm &= gm - 1u;
                        const bool b0 = u & 1, b1 = u & 2, b2 = u & 4;
                        const int cu = c0 + 4 * u;
#pragma unroll
                        for (int i = 0; i < 4; ++i) {
                            const uint32_t a0 = b0 ? v[4 + i] : v[i], a1 = b0 ? v[12 + i] : v[8 + i];
                            const uint32_t a2 = b0 ? v[20 + i] : v[16 + i], a3 = b0 ? v[28 + i] : v[24 + i];
                            const uint32_t c01 = b1 ? a1 : a0, c23 = b1 ? a3 : a2;
                            const float x = __uint_as_float(b2 ? c23 : c01);
                            if (x <= tvl && cu + i < nlim) {
                                const float xu = x * inv;
                                const float dc = (xu < 0.f) ? 0.f : xu;  // clamp
                                int slot;
                                if constexpr (PAIR > 1) slot = (int)atom_add_shared(np_s, 1u);
                                else { slot = (int)ld_vol_shared_u32(np_s); st_shared_u32(np_s, (uint32_t)slot + 1u); }
                                pool[slot] = ((unsigned long long)key_of(dc) << 32) | (colt + (uint32_t)(cu + i));
                                if (PROF) prof_app++;
                            }
                        }
                    }
                    if (PROF) { prof_rare += clock64() - cr0; prof_nrare++; }
                };
                const int cb = half * (WCOLS / 32), ce = cb + WCOLS / 32;
                if constexpr (EW >= 16) {
                    // (16 warps: TMEM load latency is short next to the warp count; one
                    // 32-register buffer keeps the epilogue within its register budget)
#pragma unroll 1
                    for (int c = cb; c < ce; ++c) {
                        uint32_t va[32];
                        tmem_ld32(taddr + (uint32_t)(c * 32), va);
                        scan32(va, c * 32);
                    }
                } else {
                    uint32_t va[32], vb[32];
                    tmem_ld32_issue(taddr + (uint32_t)(half * WCOLS), va);
                    tmem_wait32(va);
#pragma unroll 1
                    for (int c = cb; c < ce; c += 2) {
                        tmem_ld32_issue(taddr + (uint32_t)((c + 1) * 32), vb);
                        scan32(va, c * 32);
                        tmem_wait32(vb);
                        if (c + 2 < ce) tmem_ld32_issue(taddr + (uint32_t)((c + 2) * 32), va);
                        scan32(vb, (c + 1) * 32);
                        if (c + 2 < ce) tmem_wait32(va);
                    }
                }
            }
#pragma unroll 1
            for (int c = half * (WCOLS / KNN_CW); c < ((DUMP || (PIPE_ONLY && !NO_READ)) ? (half + 1) * (WCOLS / KNN_CW) : 0); ++c) {
                uint32_t v[KNN_CW];
                tmem_ld64(taddr + (uint32_t)(c * KNN_CW), v);
                if (PIPE_ONLY) {
                    if (v[0] == 0x7fc00001u && v[KNN_CW - 1] == 0x7fc00001u) st_shared_u32(np_s, 1u);  // keep the load alive
                    continue;
                }
                const int64_t col0 = (int64_t)t * BN + c * KNN_CW;
                // (knn_distances) the accumulator is d = |q|^2 + |r|^2 - 2 q.r; clamped at 0
                float d[KNN_CW];
#pragma unroll
                for (int j = 0; j < KNN_CW; ++j) d[j] = __uint_as_float(v[j]) * inv;
                if (qvalid)
                    for (int j = 0; j < KNN_CW; ++j)
                        if (col0 + j < g.N) dump[q * g.N + col0 + j] = (d[j] < 0.f) ? 0.f : d[j];
            }
            if (PROF) prof_chunks += clock64() - cc0;
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive_cta(&acce[b]);
        }
        const unsigned long long prof_t1 = PROF ? clock64() : 0;
        if (!DUMP && !PIPE_ONLY) {
            // Narrow every pool to this split's exact top-k; its k-th pair is published
            // (the bound the later splits and the merge start from).  The pool holds every
            // pair of this split in the row's top-k (all pairs <= any bound; narrowing keeps
            // the pool's k smallest); launch_merge_pools gathers the pools' pairs <= the
            // final published bound and selects the exact top-k of the row.
            narrow_lanes(g.P - g.k, g.k, g.P, true);  // n > k  <=>  n + (P - k) > P
            if (qvalid && half == 0) cnt_out[list * g.Q + q] = failed ? 0 : (int)ld_vol_shared_u32(np_s);
        }
        if (PROF) {
            __syncwarp();
            const unsigned long long prof_t2 = clock64();
            if (lane == 0) {
                unsigned long long* o = reinterpret_cast<unsigned long long*>(dump) + ((size_t)blockIdx.x * EW + e) * 16;
                o[0] = prof_narrow; o[1] = prof_wait; o[2] = prof_chunks; o[3] = prof_rare; o[4] = prof_nrare;
                o[5] = prof_nnarrow; o[6] = prof_t2 - prof_t1; o[7] = prof_t2 - prof_t0; o[8] = prof_app;
            }
        }
    }

    tc_fence_before();
    __syncthreads();
    if (g.cs > 1) cluster_sync_all();  // no peer multicasts into / arrives on this CTA any more
    tc_fence_after();
    if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(512) : "memory");
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
static size_t al256(size_t x) { return (x + 255u) & ~(size_t)255u; }

struct KnnWork {
    size_t ref_img, tscale, csum, rownorm, fix, cand, ccount, stats, q_img, qstat, pool, cnt, qthr, qspec, qfail, fb, prof, total;
};

// Queries are processed in chunks (multiples of 128 queries) so that the pools,
// lists * Qc * P * 8 bytes, stay below kPoolBudget (a k-NN graph of 10^6
// points would otherwise need tens of GB of workspace).
constexpr size_t kPoolBudget = 2ull << 30;

// sampled tiles: up to 128 (KSEL_KNN_SPEC, 0: off), at most 1/16 of the references, at
// least 8 (N >= 32768; smaller sets start cold).  C4 A/B (profiles/r02_knn_spec_size_ab.txt):
// 32 / 64 / 96 / 128 tiles -> filter 3.64 / 3.59 / 3.40 / 3.31 ms, call 4.55 / 4.59 / 4.47 / 4.48 ms
static int knn_spec_tiles(const KnnGeom& g) {
    static const int env = env_int("KSEL_KNN_SPEC", 128);
    if (env <= 0 || g.tstride != 1) return 0;
    const int ms = std::min(env, g.NT / 16);
    return ms >= 8 ? ms : 0;
}

// max_lists > 0: cap the split count so that S * halves * Q <= max_lists (a later query
// chunk must fit the workspace laid out for the first)
static KnnGeom knn_geometry(int64_t N, int64_t Q, int D, int k, int num_sms, int64_t idx_offset,
                            int64_t max_lists = 0) {
    KnnGeom g{};
    g.N = N;
    g.Q = Q;
    g.D = D;
    g.Dp = (D + KNN_KS - 1) / KNN_KS * KNN_KS;
    g.KS = g.Dp / KNN_KS;
    g.QT = (int)((Q + KNN_BM - 1) / KNN_BM);
    // two query tiles per CTA on 128-reference tiles: every reference stage feeds 256
    // queries (half the bytes landed in shared memory per distance); the pair of
    // query images must fit next to the ring (D <= 128)
#ifdef KSEL_EXPERIMENTS
    static const int qpc_env = env_int("KSEL_KNN_QPC", 1);
#else
    constexpr int qpc_env = 1;
#endif
    g.QPC = (qpc_env == 2 && g.Dp <= 128 && g.QT >= 2) ? 2 : 1;
    g.BN = (g.QPC == 2) ? 128 : 256;
    g.NT = (int)((N + g.BN - 1) / g.BN);
#ifdef KSEL_EXPERIMENTS
    static const int cs_env = [] {
        const int v = env_int("KSEL_KNN_CLUSTER", 1);  // experiments: cluster size 1, 2 or 4
        return (v == 2 || v == 4) ? v : 1;
    }();
#else
    constexpr int cs_env = 1;
#endif
    // Every CTA streams its whole reference range through L2 -> shared memory (4 B per
    // dim and reference per 128 queries): with one CTA per query tile that stream, not
    // the tensor pipe, is the floor (measured: ~40 B/clk/SM, the chip's L2 -> SM rate).
    // A cluster of cs query tiles loads each stage once (every CTA a 1/cs slice,
    // multicast to all), cutting the L2 traffic per MMA by cs.  Measured on C4: no
    // gain (cs = 1 / 2 / 4: 6.79 / 6.95 / 8.16 ms; pipeline-only 1-pass 4.08 / 4.36 /
    // 5.14 ms), so L2 is not the floor and the default is cs = 1.
    g.cs = (g.QPC == 1 && g.QT >= cs_env) ? cs_env : 1;
    g.QTp = (g.QPC == 2) ? (g.QT + 1) / 2 : (g.QT + g.cs - 1) / g.cs * g.cs;  // CTA rows of the grid
    g.k = k;
    const int kk = k < 32 ? 32 : k;
    // room for >= 1 tile of candidates after narrowing to k; register narrowing holds 1152
    // register narrowing (<= 1280 pairs) for k' <= 128; larger queues get a pool with
    // room for 8 tiles of candidates between narrowings (radix select, pool_select64)
    int P = (kk <= 128) ? 1152 : kk + 8 * 256;
    g.P = (P + 31) / 32 * 32;
    // epilogue warps: 16 (four per TMEM lane quadrant, 64 columns of every tile each) or 8;
    // result-preserving (the warps of a quadrant share each query's pool and bound)
    static const int ew_env = [] {
        const int v = env_int("KSEL_KNN_EW", 16);
#ifdef KSEL_EXPERIMENTS
        if (v == 4) return 4;
#endif
        return v == 8 ? 8 : 16;
    }();
    g.halves = (g.QPC == 2) ? 1 : ew_env / 4;
    g.EW = (g.QPC == 2) ? 8 : 4 * g.halves;
    // ring depth: as many stages as fit next to the resident query tile(s)
    const int fixed =
        1024 + g.QPC * (g.Dp * 512 + KNN_NORM_A_BYTES) + KnnSmem::scratch(g.EW, g.QPC) + 512;
    g.NS = (kMaxSmemPerBlock - fixed) / g.stage_bytes();
    if (g.NS > 12) g.NS = 12;
    g.idx_offset = idx_offset;
    static const int cap_env = env_int("KSEL_KNN_SOFTCAP", 0);  // experiments: narrow early (pool fill cap)
    // narrow before a pool reaches P when queues are small: the bound then tracks the
    // k-th of what has been seen more closely in cold CTAs (measured: 512 for k <= 128)
    const int cap = cap_env > 0 ? cap_env : (kk <= 128 ? 512 : g.P);
    g.pcap = std::max(kk + 32 + g.BN, std::min(g.P, cap));
    g.ntiles = g.NT;
    g.tstride = 1;
    // first-wave CTAs sample 16 tiles (4096 references) for their starting bound
    static const int sample_env = env_int("KSEL_KNN_SAMPLE", 16);  // experiments: tiles sampled (0 = off)
    g.sample_tiles = sample_env;
    g.sample_ctas = g.sample_tiles > 0 ? num_sms / g.cs * g.cs : 0;  // whole clusters
    // reference splits: enough CTAs for the SMs, waves as full as possible, <= 64 lists to merge
    int best = 1;
    double best_cost = 1e30;
    const int smax = (int)((g.NT < 64) ? g.NT : 64);
    for (int s = 1; s <= smax; ++s) {
        if (max_lists > 0 && s > 1 && (int64_t)s * Q > max_lists) break;
        const double ctas = (double)g.QTp * s;
        const double waves = ctas / num_sms;
        const double cost = (double)((int64_t)((ctas + num_sms - 1) / num_sms)) / waves  // tail efficiency
                            + (waves < 2.0 ? (2.0 - waves) : 0.0)                        // too few waves
                            + 0.01 * s * (kk > 128 ? kk / 128.0 : 1.0);                   // merge/pool/cold starts
        if (cost < best_cost) { best_cost = cost; best = s; }
    }
    g.S = best;
    // first-wave (cold) splits take twice the references of the others: their published
    // k-th then covers more of each query's row before the later splits start from it
    // (late r2, run_knn.py: C4 filter 6.03 -> 5.84 ms, k = 1024 13.66 -> 13.20 ms; 1.5x
    // and 2.5-4x measured worse on one of the two)
    static const int coldw_env = env_int("KSEL_KNN_COLDW", 2000);  // first-wave split weight (per mille)
    g.cold_w = (coldw_env > 0 && coldw_env <= 8000) ? coldw_env : 2000;
    static const int splits_env = env_int("KSEL_KNN_SPLITS", 0);  // experiments: force the split count
    if (splits_env > 0) {
        g.S = std::min(splits_env, smax);
        if (max_lists > 0) g.S = (int)std::max<int64_t>(1, std::min<int64_t>(g.S, max_lists / Q));
    }
    g.cold_splits = std::min(g.S, (num_sms + g.QTp - 1) / g.QTp);
    g.nstride = 1;
    g.prepass = 0;
    g.spec_ms = knn_spec_tiles(g);
    if (g.spec_ms > 0) {
        // a speculative start: no split is cold (equal splits); bounds are refreshed and
        // pools checked every 8 tiles (KSEL_KNN_NSTRIDE=4: every 4; 8 measured 3 % faster),
        // so pools get room for that many tiles of candidates beyond k + a band's worth, and
        // narrow only when that room runs out
        g.cold_splits = 0;
        g.nstride = env_int("KSEL_KNN_NSTRIDE", 8) == 4 ? 4 : 8;
        g.P = std::max(g.P, (kk + g.nstride * g.BN + 256 + 31) / 32 * 32);
        g.pcap = g.P;
    }
    return g;
}

// Speculative bounds (late r2).  With S splits per query, each split's running bound
// converges on its own 1/S of the references, so a query admits ~S k ln(N / (S k))
// candidates (C4: ~6200 per query, 60x its k) and almost every 32 x 32 epilogue chunk
// takes the rare path.  A pre-pass of the same kernel over a strided sample of m = ms x BN
// references (S = 1, target j) yields T_spec = the j-th smallest sampled d~.  The count
// of ALL references with d~ <= T_spec is ~ (N / m) Gamma(j); the verification fails when
// >= j of the k nearest fall in the sample: P = P(Poisson(lambda) >= j), lambda = k m / N.
// j = lambda + 5 sqrt(lambda) + 5 keeps it below ~1e-8 per query at C4 (128 sampled tiles:
// lambda = 3.3, j = 18); 6 sigma was measured ~1-2 % slower.  The main pass admits against T_spec from its first
// tile; knn_rescore_kernel verifies it (>= k pooled pairs <= T_spec, or a published
// bound <= T_spec), else the query takes the exact fallback -- exact either way.
static KnnGeom knn_spec_geometry(const KnnGeom& g, int ms) {
    KnnGeom p = g;
    const double lam = (double)g.k * (double)ms * g.BN / (double)g.N;
    int j = (int)std::ceil(lam + 5.0 * std::sqrt(lam) + 5.0);
    p.k = std::min(j, KNN_BN);
    const int kk = p.k < 32 ? 32 : p.k;
    const int P = (kk <= 128) ? 1152 : kk + 8 * 256;
    p.P = (P + 31) / 32 * 32;
    // narrow as soon as a tile's room is left: the running bound (cold: the first tile's
    // j-th) then tightens every few tiles instead of after ~30 (j << the sample)
    p.pcap = kk + g.BN + 128;
    p.ntiles = ms;
    p.tstride = g.NT / ms;
    p.S = 1;
    p.sample_tiles = 0;
    p.sample_ctas = 0;
    p.cold_splits = 0;
    p.nstride = 1;
    p.spec_ms = 0;
    p.prepass = 1;
    return p;
}

static KnnWork knn_work_layout(const KnnGeom& g) {
    KnnWork w{};
    size_t off = 0;
    w.ref_img = off; off += al256((size_t)g.NT * g.tile_bytes());
    w.tscale = off;  off += al256((size_t)g.NT * 8);
    w.csum = off;    off += al256((size_t)g.Dp * 24);
    w.fix = off;     off += al256((size_t)(g.NT + g.QTp * g.QPC + 1) * 4);  // [count][tiles to rebuild]
    w.rownorm = off; off += al256((size_t)(g.NT + g.QTp * g.QPC) * KNN_BN * 8);
    w.stats = off;   off += al256(sizeof(KnnStats));
    w.q_img = off;   off += al256((size_t)g.QTp * g.QPC * g.a_bytes());
    w.qstat = off;   off += al256((size_t)g.Q * 16);
    w.pool = off;    off += al256((size_t)g.S * g.Q * g.P * 8);  // one pool per (split, query)
    w.cnt = off;     off += al256((size_t)g.S * g.Q * 4);
    w.qthr = off;    off += al256((size_t)g.Q * 8);
    w.qspec = off;   off += al256((size_t)g.Q * 8);
    w.qfail = off;   off += al256((size_t)g.Q * 4);
    w.cand = off;    off += al256((size_t)g.Q * kCandCap * 8);
    w.ccount = off;  off += al256((size_t)g.Q * 4);
    w.fb = off;      off += al256(knn_fallback_bytes(g.k));
    w.prof = off;    off += al256((size_t)g.QTp * g.S * KNN_MAX_EW * 16 * 8);  // MODE 3 counters
    w.total = off;
    return w;
}

// queries per chunk (a multiple of 128, or Q), so that the pools fit kPoolBudget
static int64_t knn_query_chunk(int64_t N, int64_t Q, int D, int k, int sms) {
    int64_t qc = Q;
    for (;;) {
        const KnnGeom g = knn_geometry(N, qc, D, k, sms, 0);
        if ((size_t)g.S * (size_t)qc * (size_t)g.P * 8u <= kPoolBudget || qc <= KNN_BM) return qc;
        qc = std::max<int64_t>(KNN_BM, (qc / 2 + KNN_BM - 1) / KNN_BM * KNN_BM);
    }
}

static size_t knn_workspace_bytes(int64_t N, int64_t Q, int D, int k, int sms) {
    return knn_work_layout(knn_geometry(N, knn_query_chunk(N, Q, D, k, sms), D, k, sms, 0)).total;
}

static int knn_device_sms() {
    DevInfo di;
    return current_device_info(&di) == KSEL_OK ? di.sms : 148;
}

// knn_distances: the bound eps_q of every query (diagnostic output)
__global__ void knn_eps_kernel(const float4* __restrict__ qstat, const KnnStats* __restrict__ st, int D, int64_t Q,
                               float* __restrict__ out) {
    const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (q < Q) out[q] = knn_eps(qstat[q], *st, D);
}

// The reference image is built once per call (with the first query chunk); queries go
// in chunks of Qc, the workspace laid out for a full chunk (gq).
static cudaError_t knn_run(const float* ref, const float* query, int64_t N, int64_t Q, int D, int k,
                           int64_t idx_offset, uint8_t* work, float* out_dist, int32_t* out_idx, float* dump,
                           float* dump_eps, int sms, cudaStream_t stream) {
    const int64_t Qc = knn_query_chunk(N, Q, D, k, sms);
    const KnnGeom gq = knn_geometry(N, Qc, D, k, sms, idx_offset);
    const KnnWork w = knn_work_layout(gq);
    uint4* ref_img = reinterpret_cast<uint4*>(work + w.ref_img);
    uint4* q_img = reinterpret_cast<uint4*>(work + w.q_img);
    float4* qstat = reinterpret_cast<float4*>(work + w.qstat);
    KnnStats* stats = reinterpret_cast<KnnStats*>(work + w.stats);
    float2* tscale = reinterpret_cast<float2*>(work + w.tscale);
    double* csum = reinterpret_cast<double*>(work + w.csum);
    double* rownorm = reinterpret_cast<double*>(work + w.rownorm);
    int* fixcnt = reinterpret_cast<int*>(work + w.fix);
    int* fixlist = fixcnt + 1;
    cudaError_t e = cudaMemsetAsync(stats, 0, sizeof(KnnStats), stream);
    if (e != cudaSuccess) return e;
    for (int64_t q0 = 0; q0 < Q; q0 += Qc) {
        const int64_t nq = std::min(Qc, Q - q0);
        const KnnGeom g = knn_geometry(N, nq, D, k, sms, idx_offset, (int64_t)gq.S * Qc);
        const int nt = (q0 == 0) ? g.NT : 0;  // reference tiles: first chunk only
        if (nt > 0) {
            e = cudaMemsetAsync(csum, 0, (size_t)g.Dp * 24, stream);
            if (e != cudaSuccess) return e;
            knn_sum_kernel<<<dim3((unsigned)(g.Dp / 32), 32), 256, 0, stream>>>(ref, N, D, g.Dp, csum);
            note_launch();
        }
        e = cudaMemsetAsync(fixcnt, 0, 4, stream);
        if (e != cudaSuccess) return e;
        // one read of the points at the call's common scale; then the (rare) tiles whose
        // values exceed it rebuilt from their own max (grid-stride over the list: usually empty)
        const bool vec4 = (D & 3) == 0 && (reinterpret_cast<uintptr_t>(ref) & 15u) == 0 &&
                          (reinterpret_cast<uintptr_t>(query + q0 * (int64_t)D) & 15u) == 0;
        const size_t prep_smem = vec4 ? 0 : sizeof(float) * KNN_BN * (KNN_KS + 1);
        knn_prep1_kernel<<<(unsigned)(nt + g.QT), 256, prep_smem, stream>>>(ref, query + q0 * (int64_t)D, g, nt, csum, qstat,
                                                                    tscale, stats, ref_img, q_img, fixlist, fixcnt);
        note_launch();
        knn_stats_kernel<<<(unsigned)sms, KNN_PREP_THREADS, 0, stream>>>(
            ref, query + q0 * (int64_t)D, g, nt, csum, rownorm, qstat, tscale, stats, fixlist, fixcnt);
        note_launch();
        knn_prep_kernel<<<(unsigned)sms, KNN_PREP_THREADS, 0, stream>>>(
            ref, query + q0 * (int64_t)D, g, nt, csum, rownorm, qstat, tscale, ref_img, q_img, fixlist, fixcnt);
        note_launch();
        e = cudaGetLastError();
#ifdef KSEL_EXPERIMENTS
        // experiment: keep the previous call's final bounds (same inputs: the best bounds
        // the filter could start from -- an upper limit on what better bounds can gain;
        // profiles/r02_knn_bounds_exp.txt)
        static const bool keep_thr = env_int("KSEL_KNN_KEEPTHR", 0) == 1;
        if (!keep_thr)
#endif
        if (e == cudaSuccess) e = cudaMemsetAsync(work + w.qthr, 0xff, (size_t)nq * 8, stream);  // "no bound yet"
        if (e == cudaSuccess) e = cudaMemsetAsync(work + w.qfail, 0, (size_t)nq * 4, stream);
        if (e != cudaSuccess) return e;
        float* kdump = dump ? dump + q0 * N : nullptr;
#ifdef KSEL_EXPERIMENTS
        // Timing experiments only (a -DKSEL_EXPERIMENTS build; the product library has none of
        // these): 2 pipeline only, 3 counters, 4 no TMEM reads -- modes 2 and 4 return no result.
        static const int mode_env = [] {
            const int m = env_int("KSEL_KNN_MODE", 0);
            return (m >= 2 && m <= 4) ? m : 0;
        }();
        const int ewh = g.halves;
        auto kern = (g.QPC == 2)
                        ? (dump ? knn_fused_kernel<1, 8, 128, 2>
                           : mode_env == 2 ? knn_fused_kernel<2, 8, 128, 2>
                           : mode_env == 3 ? knn_fused_kernel<3, 8, 128, 2>
                           : mode_env == 4 ? knn_fused_kernel<4, 8, 128, 2>
                                           : knn_fused_kernel<0, 8, 128, 2>)
                    : dump ? (ewh == 4 ? knn_fused_kernel<1, 16, 256, 1> : ewh == 2 ? knn_fused_kernel<1, 8, 256, 1> : knn_fused_kernel<1, 4, 256, 1>)
                    : mode_env == 2 ? (ewh == 2 ? knn_fused_kernel<2, 8, 256, 1> : knn_fused_kernel<2, 4, 256, 1>)
                    : mode_env == 3 ? (ewh == 4 ? knn_fused_kernel<3, 16, 256, 1> : ewh == 2 ? knn_fused_kernel<3, 8, 256, 1> : knn_fused_kernel<3, 4, 256, 1>)
                    : mode_env == 4 ? knn_fused_kernel<4, 4, 256, 1>
                                    : (ewh == 4 ? knn_fused_kernel<0, 16, 256, 1> : ewh == 2 ? knn_fused_kernel<0, 8, 256, 1> : knn_fused_kernel<0, 4, 256, 1>);
        auto sel_kern = (g.QPC == 2) ? knn_fused_kernel<0, 8, 128, 2>
                                     : (ewh == 4 ? knn_fused_kernel<0, 16, 256, 1> : ewh == 2 ? knn_fused_kernel<0, 8, 256, 1> : knn_fused_kernel<0, 4, 256, 1>);
        if (!dump && mode_env == 3) kdump = reinterpret_cast<float*>(work + w.prof);
#else
        constexpr int mode_env = 0;
        const bool ew16 = g.halves == 4;
        auto kern = dump ? (ew16 ? knn_fused_kernel<1, 16, 256, 1> : knn_fused_kernel<1, 8, 256, 1>)
                         : (ew16 ? knn_fused_kernel<0, 16, 256, 1> : knn_fused_kernel<0, 8, 256, 1>);
        auto sel_kern = ew16 ? knn_fused_kernel<0, 16, 256, 1> : knn_fused_kernel<0, 8, 256, 1>;
#endif
        auto launch = [&](decltype(kern) kf, const KnnGeom& gg, unsigned long long* thr,
                          const unsigned long long* spec, float* kd, bool timed) -> cudaError_t {
            const int smem = KnnSmem::total(gg);
            cudaError_t le = ensure_smem_attr(reinterpret_cast<const void*>(kf), smem);
            if (le != cudaSuccess) return le;
            const int slot = timed ? timing_begin(stream) : -1;
            cudaLaunchConfig_t cfg{};
            cudaLaunchAttribute attr[1];
            cfg.gridDim = dim3((unsigned)(gg.QTp * gg.S));
            cfg.blockDim = dim3((unsigned)knn_threads(gg.EW));
            cfg.dynamicSmemBytes = (size_t)smem;
            cfg.stream = stream;
            attr[0].id = cudaLaunchAttributeClusterDimension;
            attr[0].val.clusterDim.x = (unsigned)gg.cs;
            attr[0].val.clusterDim.y = 1;
            attr[0].val.clusterDim.z = 1;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            le = cudaLaunchKernelEx(&cfg, kf, gg, reinterpret_cast<const uint8_t*>(ref_img),
                                    reinterpret_cast<const uint8_t*>(q_img), static_cast<const float4*>(qstat),
                                    static_cast<const KnnStats*>(stats),
                                    reinterpret_cast<unsigned long long*>(work + w.pool),
                                    reinterpret_cast<int32_t*>(work + w.cnt), thr,
                                    reinterpret_cast<int32_t*>(work + w.qfail), kd, spec, tscale);
            note_launch();
            if (timed) timing_end(slot, stream);
            return le == cudaSuccess ? cudaGetLastError() : le;
        };
        // speculative pre-pass (selection only): T_spec per query into qspec
        const int ms = (dump || mode_env != 0) ? 0 : g.spec_ms;
        unsigned long long* qspec = ms > 0 ? reinterpret_cast<unsigned long long*>(work + w.qspec) : nullptr;
        if (ms > 0) {
            e = cudaMemsetAsync(qspec, 0xff, (size_t)nq * 8, stream);
            if (e == cudaSuccess) e = launch(sel_kern, knn_spec_geometry(g, ms), qspec, nullptr, nullptr, false);
            if (e != cudaSuccess) return e;
        }
        KnnGeom gm = g;
        if (ms == 0) {  // (knn_distances / experiment modes: no speculative start)
            gm.nstride = 1;
            gm.pcap = std::min(gm.pcap, gm.P);
        }
        e = launch(kern, gm, reinterpret_cast<unsigned long long*>(work + w.qthr), qspec, kdump, !dump);
        if (e != cudaSuccess) return e;
        if (dump) {
            if (dump_eps) {
                knn_eps_kernel<<<(unsigned)((nq + 255) / 256), 256, 0, stream>>>(qstat, stats, D, nq, dump_eps + q0);
                note_launch();
                e = cudaGetLastError();
                if (e != cudaSuccess) return e;
            }
            continue;
        }
        if (mode_env == 3) continue;
        KnnRescoreArgs a{};
        a.ref = ref;
        a.query = query + q0 * (int64_t)D;
        a.N = N;
        a.Q = nq;
        a.D = D;
        a.k = k;
        a.idx_offset = idx_offset;
        a.pools = reinterpret_cast<const unsigned long long*>(work + w.pool);
        a.P = g.P;
        a.cnt = reinterpret_cast<const int32_t*>(work + w.cnt);
        a.S = g.S;
        a.thr = reinterpret_cast<const unsigned long long*>(work + w.qthr);
        a.qfail = reinterpret_cast<int32_t*>(work + w.qfail);
        a.spec = qspec;
        a.qstat = qstat;
        a.stats = stats;
        a.fb = work + w.fb;
        a.cand = reinterpret_cast<unsigned long long*>(work + w.cand);
        a.ccount = reinterpret_cast<int32_t*>(work + w.ccount);
        a.out_val = out_dist + q0 * k;
        a.out_idx = out_idx + q0 * k;
        e = launch_knn_rescore(a, stream);
        if (e == cudaSuccess) e = launch_knn_fallback(a, stream);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

static int knn_check(const float* ref, const float* query, int64_t N, int64_t Q, int D, int k, int64_t idx_offset) {
    if (!ref || !query) return KSEL_ERR_INVALID_ARG;
    if (N < 1 || Q < 1 || D < 1 || k < 1 || k > N || idx_offset < 0 || N + idx_offset > 0x7fffffffLL)
        return KSEL_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(ref) & 3u) || (reinterpret_cast<uintptr_t>(query) & 3u))
        return KSEL_ERR_INVALID_ARG;
    if (D > KNN_MAX_D || k > KSEL_MAX_K) return KSEL_ERR_UNSUPPORTED;
    return KSEL_OK;
}

// knn_graph: row i of knn_search(points, points, k + 1) without i.  One warp per
// row: find i among the k + 1 indices (ballot), copy the others in order.
__global__ void __launch_bounds__(256)
    knn_drop_self_kernel(const float* __restrict__ tv, const int32_t* __restrict__ ti, int64_t N, int k,
                         float* __restrict__ ov, int32_t* __restrict__ oi) {
    const int64_t row = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
    const uint32_t lane = lane_id();
    if (row >= N) return;
    const int k1 = k + 1;
    const float* rv = tv + row * k1;
    const int32_t* ri = ti + row * k1;
    int pos = k1;  // position of the point itself (k1: absent)
    for (int base = 0; base < k1; base += 32) {
        const int e = base + (int)lane;
        const uint32_t m = __ballot_sync(kFull, e < k1 && ri[e] == (int32_t)row);
        if (m) { pos = base + __ffs(m) - 1; break; }
    }
    for (int e = (int)lane; e < k; e += 32) {
        const int src = e < pos ? e : e + 1;
        ov[row * k + e] = rv[src];
        oi[row * k + e] = ri[src];
    }
}

}  // namespace ksel

using namespace ksel;

extern "C" {

size_t knn_search_workspace(int64_t N, int64_t Q, int D, int k) {
    if (N < 1 || Q < 1 || D < 1 || D > KNN_MAX_D || k < 1 || k > KSEL_MAX_K) return 0;
    return knn_workspace_bytes(N, Q, D, k, knn_device_sms());
}

int knn_search(const float* ref, const float* query, int64_t N, int64_t Q, int D, int k, float* out_dist,
               int32_t* out_idx, int64_t idx_offset, void* d_work, size_t work_bytes, void* stream) {
    int st = knn_check(ref, query, N, Q, D, k, idx_offset);
    if (st) return st;
    if (!out_dist || !out_idx || !d_work) return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    if (work_bytes < knn_workspace_bytes(N, Q, D, k, di.sms)) return KSEL_ERR_INVALID_ARG;
    cudaError_t e = knn_run(ref, query, N, Q, D, k, idx_offset, static_cast<uint8_t*>(d_work), out_dist, out_idx,
                            nullptr, nullptr, di.sms, (cudaStream_t)stream);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

size_t knn_graph_workspace(int64_t N, int D, int k) {
    if (N < 2 || k < 1 || k > N - 1 || k + 1 > KSEL_MAX_K) return 0;
    const size_t base = knn_search_workspace(N, N, D, k + 1);
    if (base == 0) return 0;
    return al256(base) + 2 * al256((size_t)N * (k + 1) * 4);
}

int knn_graph(const float* points, int64_t N, int D, int k, float* out_dist, int32_t* out_idx, void* d_work,
              size_t work_bytes, void* stream) {
    if (!points || !out_dist || !out_idx || N < 2 || k < 1 || k > N - 1) return KSEL_ERR_INVALID_ARG;
    int st = knn_check(points, points, N, N, D, k + 1, 0);
    if (st) return st;
    if (!d_work) return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    const size_t base = al256(knn_workspace_bytes(N, N, D, k + 1, di.sms));
    const size_t tmp = al256((size_t)N * (k + 1) * 4);
    if (work_bytes < base + 2 * tmp) return KSEL_ERR_INVALID_ARG;
    uint8_t* w = static_cast<uint8_t*>(d_work);
    float* tv = reinterpret_cast<float*>(w + base);
    int32_t* ti = reinterpret_cast<int32_t*>(w + base + tmp);
    cudaError_t e = knn_run(points, points, N, N, D, k + 1, 0, w, tv, ti, nullptr, nullptr, di.sms,
                            (cudaStream_t)stream);
    if (e != cudaSuccess) return KSEL_ERR_CUDA;
    knn_drop_self_kernel<<<(unsigned)((N + 7) / 8), 256, 0, (cudaStream_t)stream>>>(tv, ti, N, k, out_dist, out_idx);
    note_launch();
    return cudaGetLastError() == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

size_t knn_distances_workspace(int64_t N, int64_t Q, int D) { return knn_search_workspace(N, Q, D, 1); }

int knn_distances(const float* ref, const float* query, int64_t N, int64_t Q, int D, float* out, float* out_eps,
                  void* d_work, size_t work_bytes, void* stream) {
    int st = knn_check(ref, query, N, Q, D, 1, 0);
    if (st) return st;
    if (!out || !d_work) return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    if (work_bytes < knn_workspace_bytes(N, Q, D, 1, di.sms)) return KSEL_ERR_INVALID_ARG;
    cudaError_t e = knn_run(ref, query, N, Q, D, 1, 0, static_cast<uint8_t*>(d_work), nullptr, nullptr, out, out_eps,
                            di.sms, (cudaStream_t)stream);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

}  // extern "C"
