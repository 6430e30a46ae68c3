// select_radix.cu -- KSEL_ALGO_RADIX: ksel_select for rows of up to 65536 values,
// a cluster of CTAs per row, the row held in registers, exact radix narrowing
// of the k-th key across the cluster (the value-bucket form
// of the paper's Hierarchical Partition), then one sort.
//
// An alternative to the streaming pool kernel (select_pool.cu, the default):
// its cost does not depend on the value order (sorted, tied and random rows
// cost the same) and barely on k.  Measured on C2 (Q = 1024, N = 65536) it is
// slower than the pool kernel except for heavy ties at k = 1024 (U: 0.21 ms at
// k = 1, 0.48 ms at k = 1024 vs 0.08 / 0.41 ms; T k = 1024: 0.54 vs 0.56 ms):
// the per-pass barriers (CTA and cluster) and the sort leave the SMs idle
// between waves of loads (ncu: 36 % of stalls on barriers).  Kept as the
// exact value-bucket (HP) variant; ksel_select's automatic choice is the pool
// kernel.
//
// Per row r, a cluster of CS = ceil(N / 8192) CTAs (<= 8); CTA j holds the
// segment [j * seg, min(N, (j + 1) * seg)) (seg = ceil(N / CS) rounded up to 4)
// as 32 order keys per thread (256 threads, 128-bit streaming loads):
//
//   up to 4 passes of 8 bits, most significant first (value buckets, L225):
//     every CTA histograms the current digit of the keys that share the known
//     prefix (per-warp shared-memory histograms, summed per CTA);
//     cluster barrier; every CTA reads all CTAs' histograms (DSMEM) and finds
//     the same bucket b holding the remaining rank; keys below b's range are
//     certainly selected, above certainly not (the guarantee of L225, exact
//     because buckets are ordered by value);
//     once the certain keys plus the bucket fit CTA 0's 2048-pair buffer, all
//     of them are sent (bucket mode) and the sort decides;
//   else, after pass 4, v* = the exact k-th smallest key and `need` = ties of
//   v* to take: CTA j selects its keys < v*, plus its share of the ties in
//   index order (CTA order = index order, so the quota of CTA j is what the
//   lower ranks leave; inside a CTA ties are ranked by block scans in index
//   order) -- reading R1 (lexicographic (value, index));
//   the selected (key, index) pairs go to CTA 0's shared memory (DSMEM stores
//   at offsets every CTA computes from the histograms), cluster barrier,
//   CTA 0 sorts them (shared-memory bitonic network) and writes the first k:
//   ascending (value, index), original value bits (-0.0 / NaN payloads, whose
//   canonical key dropped the bits, are re-read from the row).
#include <cstdint>

#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_common.cuh"
#include "ksel_internal.h"

namespace ksel {

constexpr int RX_THREADS = 256;
constexpr int RX_WARPS = RX_THREADS / 32;
constexpr int RX_EPT = 32;                     // keys per thread
constexpr int RX_G = RX_EPT / 4;               // float4 groups per thread
constexpr int RX_SEG = RX_THREADS * RX_EPT;    // 8192 values per CTA
constexpr int RX_MAX_CS = 8;                   // portable cluster size -> N <= 65536
constexpr int RX_CAND = 2048;                  // CTA 0's (key, idx) candidate buffer (>= KSEL_MAX_K)

struct RadixSmem {
    uint32_t whist[RX_WARPS][256];  // per-warp histograms of one pass
    uint32_t chist[2][256];         // the CTA's histogram (read by the whole cluster), double-buffered
    uint32_t okey[RX_CAND];         // CTA 0: the candidates (>= k), then sorted
    uint32_t oidx[RX_CAND];
    uint32_t scan[RX_WARPS + 1];
    uint32_t less[RX_MAX_CS];       // keys below the final bucket, per CTA of the cluster
    uint32_t eq[RX_MAX_CS];         // keys equal to v*, per CTA
    uint32_t sel_b, sel_excl, sel_cnt;
};

__device__ __forceinline__ uint32_t rx_cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t rx_cluster_size() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void rx_cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cluster address of `p` (this CTA's shared memory) in CTA `rank`
__device__ __forceinline__ uint32_t rx_mapa(const void* p, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_u32(p)), "r"(rank));
    return r;
}
__device__ __forceinline__ uint32_t rx_ld_cluster(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
    return v;
}
// cnt[j] = the u32 at `p`'s offset in CTA j, for j < cs (0 beyond): one asm block,
// so the eight DSMEM loads are in flight together
__device__ __forceinline__ void rx_ld_cluster8(const void* p, uint32_t cs, uint32_t (&cnt)[RX_MAX_CS]) {
    uint32_t ad[RX_MAX_CS];
#pragma unroll
    for (int j = 0; j < RX_MAX_CS; ++j) ad[j] = rx_mapa(p, (uint32_t)j < cs ? (uint32_t)j : 0u);
    asm volatile(
        "ld.shared::cluster.u32 %0, [%8];\n\tld.shared::cluster.u32 %1, [%9];\n\t"
        "ld.shared::cluster.u32 %2, [%10];\n\tld.shared::cluster.u32 %3, [%11];\n\t"
        "ld.shared::cluster.u32 %4, [%12];\n\tld.shared::cluster.u32 %5, [%13];\n\t"
        "ld.shared::cluster.u32 %6, [%14];\n\tld.shared::cluster.u32 %7, [%15];"
        : "=r"(cnt[0]), "=r"(cnt[1]), "=r"(cnt[2]), "=r"(cnt[3]), "=r"(cnt[4]), "=r"(cnt[5]), "=r"(cnt[6]),
          "=r"(cnt[7])
        : "r"(ad[0]), "r"(ad[1]), "r"(ad[2]), "r"(ad[3]), "r"(ad[4]), "r"(ad[5]), "r"(ad[6]), "r"(ad[7])
        : "memory");
#pragma unroll
    for (int j = 1; j < RX_MAX_CS; ++j) cnt[j] = ((uint32_t)j < cs) ? cnt[j] : 0u;
}
__device__ __forceinline__ void rx_st_cluster(uint32_t addr, uint32_t v) {
    asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}

// Block-wide exclusive scan of one u32 per thread (256 threads, thread order).
__device__ __forceinline__ uint32_t rx_block_excl_scan(uint32_t v, uint32_t* scan, uint32_t& total) {
    const uint32_t lane = lane_id();
    const int w = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, x, d);
        if (lane >= (uint32_t)d) x += t;
    }
    if (lane == 31) scan[w] = x;
    __syncthreads();
    if (w == 0) {
        uint32_t s = (lane < (uint32_t)RX_WARPS) ? scan[lane] : 0u;
#pragma unroll
        for (int d = 1; d < RX_WARPS; d <<= 1) {
            const uint32_t t = __shfl_up_sync(kFull, s, d);
            if (lane >= (uint32_t)d) s += t;
        }
        if (lane < (uint32_t)RX_WARPS) scan[lane] = s;  // inclusive warp totals
    }
    __syncthreads();
    total = scan[RX_WARPS - 1];
    const uint32_t base = (w > 0) ? scan[w - 1] : 0u;
    __syncthreads();  // scan[] may be reused right after
    return base + x - v;
}

template <bool VEC>
__global__ void __launch_bounds__(RX_THREADS, 4)
    ksel_radix_kernel(const float* __restrict__ dist, int64_t Q, int64_t N, int k, int64_t seg,
                      float* __restrict__ out_val, int32_t* __restrict__ out_idx) {
    __shared__ RadixSmem sm;
    const uint32_t cs = rx_cluster_size();
    const uint32_t rank = rx_cluster_rank();
    const int64_t row = blockIdx.x / cs;
    const int t = threadIdx.x;
    const int w = t >> 5;
    const uint32_t lane = lane_id();
    const int64_t a = (int64_t)rank * seg;
    const int len = (int)max((int64_t)0, min(N, a + seg) - a);  // keys of this CTA (<= 8192)
    const float* rowp = dist + row * N;
    const float* src = rowp + a;

    // ---- load: position p = 1024 g + 4 t + c (index order: g, then t, then c) ----
    uint32_t key[RX_EPT];
#pragma unroll
    for (int g = 0; g < RX_G; ++g) {
        const int p = g * (RX_THREADS * 4) + 4 * t;
        if (VEC && p + 3 < len) {
            const float4 v = __ldcs(reinterpret_cast<const float4*>(src + p));
            key[4 * g + 0] = key_of(v.x);
            key[4 * g + 1] = key_of(v.y);
            key[4 * g + 2] = key_of(v.z);
            key[4 * g + 3] = key_of(v.w);
        } else {
#pragma unroll
            for (int c = 0; c < 4; ++c) key[4 * g + c] = (p + c < len) ? key_of(__ldcs(src + p + c)) : 0u;
        }
    }
    auto valid = [&](int e) { return (e >> 2) * (RX_THREADS * 4) + 4 * t + (e & 3) < len; };

    // ---- radix passes of 8 bits over the cluster's keys (at most 4) ----
    // After each pass: keys whose top bits are below the chosen bucket are certainly
    // selected, above certainly not.  As soon as the certain ones plus the bucket fit
    // CTA 0's buffer (RX_CAND pairs), every CTA sends exactly those (bucket mode) and
    // CTA 0's sort picks the first k -- typically after 1-2 passes.  Otherwise, after
    // the 4th pass the bucket is the tie class of v* = the exact k-th key: quota mode.
    uint32_t pval = 0, pmask = 0, krem = (uint32_t)k;
    bool bucket_mode = false;
    if (t < RX_MAX_CS) sm.less[t] = 0;
#pragma unroll 1
    for (int pass = 0; pass < 4; ++pass) {
        const int shift = 24 - 8 * pass;
#pragma unroll
        for (int j = 0; j < RX_WARPS; ++j) sm.whist[j][t] = 0;
        __syncthreads();
        const uint32_t hs = smem_u32(&sm.whist[w][0]);
#pragma unroll
        for (int e = 0; e < RX_EPT; ++e)
            if (valid(e) && (key[e] & pmask) == pval)
                asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(hs + ((key[e] >> shift) & 255u) * 4u) : "memory");
        __syncthreads();
        uint32_t s = 0;
#pragma unroll
        for (int j = 0; j < RX_WARPS; ++j) s += sm.whist[j][t];
        sm.chist[pass & 1][t] = s;
        rx_cluster_sync();  // every CTA's histogram of this pass is complete
        uint32_t cnt[RX_MAX_CS];
        rx_ld_cluster8(&sm.chist[pass & 1][t], cs, cnt);  // bin t of every CTA (8 loads in flight)
        uint32_t tot = 0;
#pragma unroll
        for (int j = 0; j < RX_MAX_CS; ++j) tot += cnt[j];
        uint32_t total;
        const uint32_t excl = rx_block_excl_scan(tot, sm.scan, total);
        if (excl < krem && excl + tot >= krem) {  // the bucket holding the remaining rank (unique)
            sm.sel_b = (uint32_t)t;
            sm.sel_excl = excl;
            sm.sel_cnt = tot;
#pragma unroll
            for (int j = 0; j < RX_MAX_CS; ++j) sm.eq[j] = cnt[j];
        }
        __syncthreads();
        const uint32_t b = sm.sel_b;
        krem -= sm.sel_excl;
        // per-CTA counts below the bucket (certainly selected)
#pragma unroll
        for (int j = 0; j < RX_MAX_CS; ++j) {
            uint32_t x = ((uint32_t)t < b) ? cnt[j] : 0u;
            x = __reduce_add_sync(kFull, x);
            if (lane == 0 && x) atomicAdd(&sm.less[j], x);
        }
        pval |= b << shift;
        pmask |= 255u << shift;
        const bool fits = (uint32_t)k - krem + sm.sel_cnt <= (uint32_t)RX_CAND;
        __syncthreads();
        if (fits) {
            bucket_mode = true;
            break;
        }
    }
    // bucket mode: CTA j sends less[j] + eq[j] pairs (all keys with top bits <= the
    // bucket's); quota mode: pval = v*, krem = ties of v* to take, CTA j takes the
    // first ones in index order that the lower ranks leave (reading R1)
    const uint32_t vstar = pval;
    uint32_t off = 0, quota = 0, before = 0, ncand = 0;
    for (uint32_t j = 0; j < cs; ++j) {
        const uint32_t eqj = sm.eq[j];
        const uint32_t left = (krem > before) ? krem - before : 0u;
        const uint32_t qj = bucket_mode ? eqj : (eqj < left ? eqj : left);
        if (j == rank) quota = qj;
        if (j < rank) off += sm.less[j] + qj;
        ncand += sm.less[j] + qj;
        before += eqj;
    }
    const uint32_t myeq = sm.eq[rank];

    // ---- emit this CTA's selected pairs into CTA 0's buffer ----
    uint32_t tie_rank_base[RX_G];  // rank (in index order) of this thread's first tie of group g
    const bool partial = !bucket_mode && quota > 0 && quota < myeq;
    if (partial) {  // ties cut inside this CTA: rank them in index order
        uint32_t run = 0;
#pragma unroll
        for (int g = 0; g < RX_G; ++g) {
            uint32_t c = 0;
#pragma unroll
            for (int cc = 0; cc < 4; ++cc) c += (valid(4 * g + cc) && key[4 * g + cc] == vstar) ? 1u : 0u;
            uint32_t tot;
            tie_rank_base[g] = run + rx_block_excl_scan(c, sm.scan, tot);
            run += tot;
        }
    }
    uint32_t nsel = 0;
    uint32_t selmask = 0;
#pragma unroll
    for (int g = 0; g < RX_G; ++g) {
        uint32_t tr = partial ? tie_rank_base[g] : 0u;
#pragma unroll
        for (int cc = 0; cc < 4; ++cc) {
            const int e = 4 * g + cc;
            bool sel = false;
            if (valid(e)) {
                if (bucket_mode) {
                    sel = (key[e] & pmask) <= pval;
                } else if (key[e] < vstar) {
                    sel = true;
                } else if (key[e] == vstar) {
                    sel = partial ? (tr < quota) : (quota > 0);
                    ++tr;
                }
            }
            selmask |= (sel ? 1u : 0u) << e;
            nsel += sel ? 1u : 0u;
        }
    }
    uint32_t ntot;
    uint32_t slot = off + rx_block_excl_scan(nsel, sm.scan, ntot);
    const uint32_t kdst = rx_mapa(&sm.okey[0], 0u), idst = rx_mapa(&sm.oidx[0], 0u);
#pragma unroll
    for (int e = 0; e < RX_EPT; ++e) {
        if (selmask & (1u << e)) {
            const uint32_t p = (uint32_t)((e >> 2) * (RX_THREADS * 4) + 4 * t + (e & 3));
            rx_st_cluster(kdst + slot * 4u, key[e]);
            rx_st_cluster(idst + slot * 4u, (uint32_t)(a + p));
            ++slot;
        }
    }
    rx_cluster_sync();  // CTA 0 holds all ncand (>= k) pairs; the other CTAs are done
    if (rank != 0) return;

    // ---- CTA 0: bitonic sort of the candidates (padded to a power of 2), emit k ----
    int n = 32;
    while (n < (int)ncand) n <<= 1;
    for (int e = (int)ncand + t; e < n; e += RX_THREADS) {
        sm.okey[e] = kSentKey;
        sm.oidx[e] = kSentIdx;
    }
    __syncthreads();
    for (int size = 2; size <= n; size <<= 1) {
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int i = t; i < (n >> 1); i += RX_THREADS) {
                const int lo = 2 * stride * (i / stride) + (i % stride), hi = lo + stride;
                const bool asc = (lo & size) == 0;
                const uint32_t k0 = sm.okey[lo], i0 = sm.oidx[lo], k1 = sm.okey[hi], i1 = sm.oidx[hi];
                if (pair_lt(k1, i1, k0, i0) == asc) {
                    sm.okey[lo] = k1; sm.oidx[lo] = i1;
                    sm.okey[hi] = k0; sm.oidx[hi] = i0;
                }
            }
            __syncthreads();
        }
    }
    float* ov = out_val + row * (int64_t)k;
    int32_t* oi = out_idx + row * (int64_t)k;
    for (int e = t; e < k; e += RX_THREADS) {
        const uint32_t kk = sm.okey[e], ii = sm.oidx[e];
        // -0.0 and NaN payloads: the canonical key dropped the bits -> the row's own bits
        const uint32_t bits = key_needs_regather(kk) ? __float_as_uint(rowp[ii]) : bits_of_key(kk);
        ov[e] = __uint_as_float(bits);
        oi[e] = (int32_t)ii;
    }
}

bool radix_supported(int64_t N, int k) { return N <= (int64_t)RX_SEG * RX_MAX_CS && k <= KSEL_MAX_K; }

cudaError_t launch_select_radix(const float* dist, int64_t Q, int64_t N, int k, float* ov, int32_t* oi,
                                cudaStream_t stream) {
    if (!radix_supported(N, k)) return cudaErrorInvalidValue;
    const int cs = (int)((N + RX_SEG - 1) / RX_SEG);
    int64_t seg = (N + cs - 1) / cs;
    seg = (seg + 3) / 4 * 4;  // CTA segments start 16-B aligned when the row does
    const bool vec = (N % 4 == 0) && ((reinterpret_cast<uintptr_t>(dist) & 15u) == 0);
    cudaLaunchConfig_t cfg{};
    cudaLaunchAttribute attr[1];
    cfg.gridDim = dim3((unsigned)(Q * cs));
    cfg.blockDim = dim3(RX_THREADS);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = stream;
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = vec ? cudaLaunchKernelEx(&cfg, ksel_radix_kernel<true>, dist, Q, N, k, seg, ov, oi)
                        : cudaLaunchKernelEx(&cfg, ksel_radix_kernel<false>, dist, Q, N, k, seg, ov, oi);
    note_launch();
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

}  // namespace ksel
