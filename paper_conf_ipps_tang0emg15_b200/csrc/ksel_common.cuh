// ksel_common.cuh -- device primitives shared by the sm_100a kernels of libksel.
//
// * order keys (fp32 -> ordered u32 with -0.0/NaN canonicalised), R3-R5;
// * warp-distributed sorted arrays of (key, idx) pairs and the bitonic networks
//   over them (Fig. 2 "Bitonic Merge" / "Reverse Bitonic
//   Merge"; the "flip" stage is the reverse merge's cross-compare);
// * mbarrier + cp.async.bulk (TMA bulk copy) helpers for the streaming stage.
//
// Layout of a warp array with R registers per lane: element e = r*32 + lane
// lives in register r of lane `lane`.  Strides >= 32 are in-register
// compare-exchanges, strides < 32 use __shfl_xor_sync.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ksel {

constexpr unsigned kFull = 0xffffffffu;
constexpr uint32_t kSentKey = 0xffffffffu;  // sentinel pair (kSentKey, kSentIdx) is
constexpr uint32_t kSentIdx = 0x7fffffffu;  // greater than every real pair (idx < 2^31-1)

// fp32 bits -> order-preserving u32 key.  -0.0 and +0.0 map to the same key
// (0x80000000), every NaN maps to 0xffffffff (above +Inf = 0xff800000).
__device__ __forceinline__ uint32_t key_of_bits(uint32_t b) {
    const uint32_t mag = b & 0x7fffffffu;
    uint32_t key = b ^ ((uint32_t)((int32_t)b >> 31) | 0x80000000u);
    key = (mag == 0u) ? 0x80000000u : key;
    key = (mag > 0x7f800000u) ? 0xffffffffu : key;
    return key;
}
__device__ __forceinline__ uint32_t key_of(float x) { return key_of_bits(__float_as_uint(x)); }

// Inverse of key_of_bits for every non-canonicalised key (all values except
// -0.0 and NaN payloads, which callers re-gather from the input).
__device__ __forceinline__ uint32_t bits_of_key(uint32_t key) {
    return (key & 0x80000000u) ? (key & 0x7fffffffu) : ~key;
}
__device__ __forceinline__ bool key_needs_regather(uint32_t key) {
    return key == 0x80000000u || key == 0xffffffffu;
}

// Lexicographic (key, idx) "strictly before".
// As one 64-bit unsigned compare of (key << 32 | idx): two ISETPs instead of three
// or four instructions.
__device__ __forceinline__ bool pair_lt(uint32_t ka, uint32_t ia, uint32_t kb, uint32_t ib) {
    return (((uint64_t)ka << 32) | ia) < (((uint64_t)kb << 32) | ib);
}

__device__ __forceinline__ uint32_t lane_id() {
    uint32_t l;
    asm volatile("mov.u32 %0, %%laneid;" : "=r"(l));
    return l;
}
__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// ---------------------------------------------------------------------------
// Warp-distributed arrays and bitonic networks
// ---------------------------------------------------------------------------
template <int R>
struct WArr {
    uint32_t k[R];
    uint32_t i[R];
};

template <int R>
__device__ __forceinline__ void warr_fill_sentinel(WArr<R>& a) {
#pragma unroll
    for (int r = 0; r < R; ++r) { a.k[r] = kSentKey; a.i[r] = kSentIdx; }
}

// In-register compare-exchange: lower position gets the smaller pair when asc.
// (One comparison: when descending, equal pairs are swapped too -- harmless, since
// equal pairs are identical; (key, idx) pairs are distinct except sentinels.)
__device__ __forceinline__ void cx_reg(uint32_t& ka, uint32_t& ia, uint32_t& kb, uint32_t& ib, bool asc) {
    const bool swap = pair_lt(kb, ib, ka, ia) == asc;
    const uint32_t tk = ka, ti = ia;
    ka = swap ? kb : ka; ia = swap ? ib : ia;
    kb = swap ? tk : kb; ib = swap ? ti : ib;
}

// Cross-lane compare-exchange at lane stride s: this lane keeps the min when
// `keep_min`, else the max, of (own, partner).
__device__ __forceinline__ void cx_lane(uint32_t& k, uint32_t& i, int s, bool keep_min) {
    const uint32_t ok = __shfl_xor_sync(kFull, k, s);
    const uint32_t oi = __shfl_xor_sync(kFull, i, s);
    // one comparison for both directions (the max side also takes an equal partner: identical)
    const bool take = pair_lt(ok, oi, k, i) == keep_min;
    k = take ? ok : k;
    i = take ? oi : i;
}

// In-register bitonic stage (stride s >= 32, compile time) of the network
// whose direction is set by bit m of the element position (m = 0: ascending).
template <int R, int s>
__device__ __forceinline__ void reg_stage(WArr<R>& a, int m) {
    constexpr int rs = s >> 5;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        if ((r & rs) == 0) {
            // direction from bit m of the position r*32+lane (m > s >= 32: a register bit)
            const bool asc = (m == 0) ? true : (((r << 5) & m) == 0);
            cx_reg(a.k[r], a.i[r], a.k[r | rs], a.i[r | rs], asc);
        }
    }
}

// Cross-lane stages s_hi, s_hi/2, ..., 1 (s_hi <= 16).  Kept as a runtime loop:
// the body is the same for every stride, which keeps the code (and ptxas time)
// small for large queues; the register index stays compile-time.
template <int R>
__device__ __forceinline__ void lane_stages(WArr<R>& a, int s_hi, int m, uint32_t lane) {
#pragma unroll 1
    for (int s = s_hi; s >= 1; s >>= 1) {
        const bool lower = (lane & (uint32_t)s) == 0u;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const bool asc = (m == 0) ? true : (((m >= 32) ? ((r << 5) & m) : (int)(lane & (uint32_t)m)) == 0);
            cx_lane(a.k[r], a.i[r], s, lower == asc);
        }
    }
}

template <int R, int s>
__device__ __forceinline__ void reg_stages_from(WArr<R>& a, int m) {
    if constexpr (s >= 32) {
        reg_stage<R, s>(a, m);
        reg_stages_from<R, (s >> 1)>(a, m);
    }
}

template <int R, int M>
__device__ __forceinline__ void sort_levels_from(WArr<R>& a, uint32_t lane) {
    if constexpr (M <= 32 * R) {
        const int dirbit = (M == 32 * R) ? 0 : M;
        reg_stages_from<R, (M >> 1)>(a, dirbit);
        lane_stages<R>(a, 16, dirbit, lane);
        sort_levels_from<R, (M << 1)>(a, lane);
    }
}

// Full bitonic sort, ascending, of the 32*R elements.
template <int R>
__device__ __forceinline__ void warr_sort(WArr<R>& a, uint32_t lane) {
    // levels whose blocks fit inside a warp (m <= 32): cross-lane stages only
#pragma unroll 1
    for (int m = 2; m <= 32; m <<= 1) lane_stages<R>(a, m >> 1, (m == 32 * R) ? 0 : m, lane);
    sort_levels_from<R, 64>(a, lane);
}

// Bitonic clean: sorts ascending a bitonic sequence of 32*R elements.
template <int R>
__device__ __forceinline__ void warr_clean(WArr<R>& a, uint32_t lane) {
    reg_stages_from<R, 16 * R>(a, 0);
    lane_stages<R>(a, 16, 0, lane);
}

// Keep the 32*R smallest of (q ∪ b); q and b sorted ascending (b has 32*RB
// elements, RB may differ from R).  "Flip" stage of the Reverse Bitonic Merge
// (PAPER.md L139): q[p] = min(q[p], b[L-1-p']) over the overlapping tail,
// which leaves a bitonic sequence holding exactly the 32*R smallest, then a
// bitonic clean.  The Merge Queue's lazy update is that this
// runs only when a buffer flushes.
template <int R, int RB>
__device__ __forceinline__ void warr_merge(WArr<R>& q, const WArr<RB>& b, uint32_t lane) {
    constexpr int RE = (RB < R) ? RB : R;
#pragma unroll
    for (int t = 0; t < RE; ++t) {
        const int qr = R - RE + t;
        const int br = RE - 1 - t;
        const uint32_t bk = __shfl_xor_sync(kFull, b.k[br], 31);
        const uint32_t bi = __shfl_xor_sync(kFull, b.i[br], 31);
        const bool take = pair_lt(bk, bi, q.k[qr], q.i[qr]);
        q.k[qr] = take ? bk : q.k[qr];
        q.i[qr] = take ? bi : q.i[qr];
    }
    warr_clean<R>(q, lane);
}

// x[j] for a runtime j in [0, 16): a 4-level select tree (registers cannot be indexed
// dynamically without a local-memory copy).
__device__ __forceinline__ float sel16(const float (&x)[16], int j) {
    const bool b0 = j & 1, b1 = j & 2, b2 = j & 4, b3 = j & 8;
    float l1[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) l1[i] = b0 ? x[2 * i + 1] : x[2 * i];
    float l2[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) l2[i] = b1 ? l1[2 * i + 1] : l1[2 * i];
    const float l3a = b2 ? l2[1] : l2[0], l3b = b2 ? l2[3] : l2[2];
    return b3 ? l3b : l3a;
}

// Pair at (0-based) position pos of a warp array, broadcast to all lanes.
template <int R>
__device__ __forceinline__ void warr_get(const WArr<R>& a, int pos, uint32_t& k, uint32_t& i) {
    const int rr = pos >> 5;
    uint32_t tk = 0, ti = 0;
#pragma unroll
    for (int r = 0; r < R; ++r)
        if (r == rr) { tk = a.k[r]; ti = a.i[r]; }
    k = __shfl_sync(kFull, tk, pos & 31);
    i = __shfl_sync(kFull, ti, pos & 31);
}

// Device-side flag waits (ksel_flag_wait, ksel_merge_lists) give up after a timeout
// (a kernel parameter) and record it in a mapped host word instead of hanging or
// trapping (a trap would kill the context; ksel_device_status reports it).
__device__ __forceinline__ void note_timeout(uint32_t* err) {
    if (err) {
        atomicOr(err, 1u);
        __threadfence_system();
    }
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// ---------------------------------------------------------------------------
// mbarrier / bulk async copy (TMA non-tensor) helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// min of three floats in one instruction (sm_100: FMNMX3); a NaN operand is ignored like fminf
__device__ __forceinline__ float fmin3f(float a, float b, float c) {
    float r;
    asm("min.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
    return r;
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive_cta(uint64_t* bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}
// Wait with a suspend-time hint: the waiting thread sleeps in the barrier unit
// instead of re-issuing try_wait, leaving issue slots of its SM sub-partition to
// the warps doing work (the kNN producer and MMA threads share sub-partitions
// with epilogue warps).
__device__ __forceinline__ bool mbar_try_wait_sleep(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait_sleep(bar, parity)) {
    }
}
// 1-D bulk copy global -> shared, completion signalled on `bar` (complete_tx).
// dst/src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

}  // namespace ksel
