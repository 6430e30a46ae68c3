// ksel_pool.cuh -- warp-cooperative candidate-pool primitives (radix narrowing).
//
// A "pool" is an unordered array of (key, idx) pairs (keys and indices in two
// arrays, shared or global memory).  pool_kth finds the exact want-th smallest
// pair with an MSD radix-histogram select (8-bit digits of the key, then of the
// index for ties); pool_compact keeps the pairs <= a threshold.  Together they
// are the value-bucket form of the paper's Hierarchical Partition
// (PAPER.md L221-L231): every bucket above the one holding the k-th pair is
// discarded as a whole.  Used by select_pool.cu (per-warp pools in shared
// memory) and knn_fused.cu (per-query pools in global memory).
#pragma once
#include <cstdint>

#include "ksel_common.cuh"

namespace ksel {

// Exclusive warp prefix sum of v; total in `total`.
__device__ __forceinline__ uint32_t warp_excl_scan(uint32_t v, uint32_t lane, uint32_t& total) {
    uint32_t inc = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t t = __shfl_up_sync(kFull, inc, d);
        if (lane >= (uint32_t)d) inc += t;
    }
    total = __shfl_sync(kFull, inc, 31);
    return inc - v;
}

// Histogram bins are stored transposed (bin b at (b & 7) * 32 + (b >> 3)) so
// that lane l reading its 8 bins 8l..8l+7 hits 8 distinct banks per access.
__device__ __forceinline__ int hist_slot(uint32_t b) { return (int)((b & 7u) * 32u + (b >> 3)); }

// Locate the bucket holding the want-th (1-based) element from a filled
// histogram: returns the digit; `want` becomes the rank inside that bucket and
// `cnt` the bucket's population.
__device__ __forceinline__ uint32_t hist_find(const uint32_t* hist, uint32_t lane, uint32_t& want, uint32_t& cnt) {
    uint32_t h[8], s = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        h[j] = hist[j * 32 + lane];
        s += h[j];
    }
    uint32_t total;
    const uint32_t excl = warp_excl_scan(s, lane, total);
    const bool mine = excl < want && want <= excl + s;
    const uint32_t bal = __ballot_sync(kFull, mine);
    const int src = __ffs(bal) - 1;
    uint32_t d = 0, before = excl, c = 0;
    if (mine) {
        uint32_t acc = excl;
        bool done = false;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            if (!done && acc + h[j] >= want) {
                d = lane * 8u + (uint32_t)j;
                before = acc;
                c = h[j];
                done = true;
            }
            acc += h[j];
        }
    }
    d = __shfl_sync(kFull, d, src);
    before = __shfl_sync(kFull, before, src);
    cnt = __shfl_sync(kFull, c, src);
    want -= before;
    return d;
}

// Exact want-th smallest (key, idx) pair among pool[0..n), want in [1, n].
// MSD radix select, 8-bit digits: 4 passes over the key, then (only if the
// k-th key value is tied beyond the rank needed) 4 passes over the index.
// slack > 0: stop after the first key digit whose bucket, with everything below it, holds
// at most want + slack pairs, and return (that bucket's last key, 0x7ffffffe): a valid
// (>= want pairs at or below it) but not exact bound, for mid-stream narrowings.
__device__ __noinline__ static unsigned long long pool_kth(const uint32_t* __restrict__ pk, const uint32_t* __restrict__ pi,
                                                    int n, uint32_t want, uint32_t* __restrict__ hist,
                                                    uint32_t* ties_out = nullptr, uint32_t slack = 0) {
    const uint32_t lane = lane_id();
    const uint32_t want0 = want;
    // Digits above the highest bit where the pool's smallest and largest keys differ
    // are common to all keys: start at the pass holding that bit (pools of keys near
    // one bound usually share their top byte or two).
    uint32_t kmin = 0xffffffffu, kmax = 0u;
    for (int e = (int)lane; e < n; e += 32) {
        const uint32_t key = pk[e];
        kmin = min(kmin, key);
        kmax = max(kmax, key);
    }
    kmin = __reduce_min_sync(kFull, kmin);
    kmax = __reduce_max_sync(kFull, kmax);
    uint32_t prefix = 0, cnt = (uint32_t)n;
    int first = 4;  // all keys equal: no pass, the k-th key is kmin and every key ties
    if (kmin != kmax) {
        first = __clz(kmin ^ kmax) >> 3;
        prefix = first ? (kmin & (0xffffffffu << (32 - 8 * first))) : 0u;
    } else {
        prefix = kmin;
    }
#pragma unroll 1
    for (int pass = first; pass < 4; ++pass) {
        const int shift = 24 - 8 * pass;
#pragma unroll
        for (int j = 0; j < 8; ++j) hist[j * 32 + lane] = 0u;
        __syncwarp();
#pragma unroll 4
        for (int e = (int)lane; e < n; e += 32) {
            const uint32_t key = pk[e];
            const bool sel = (pass == first) || ((key ^ prefix) >> (shift + 8)) == 0u;
            if (sel) atomicAdd(&hist[hist_slot((key >> shift) & 255u)], 1u);
        }
        __syncwarp();
        const uint32_t d = hist_find(hist, lane, want, cnt);
        prefix |= d << shift;
        __syncwarp();
        if (slack && shift > 0 && (want0 - want) + cnt <= want0 + slack) {  // take the whole bucket
            if (ties_out) *ties_out = 0;
            return ((unsigned long long)(prefix | ((1u << shift) - 1u)) << 32) | 0x7ffffffeu;
        }
    }
    const uint32_t vkey = prefix;
    if (ties_out) *ties_out = cnt;  // pool entries whose key equals the k-th key
    uint32_t idx;
    if (cnt == want) {
        // every tie of the k-th key is needed: the threshold is the largest such index
        uint32_t m = 0;
        for (int e = (int)lane; e < n; e += 32)
            if (pk[e] == vkey) m = max(m, pi[e]);
        idx = __reduce_max_sync(kFull, m);
    } else {
        // the same prefix skip over the tied keys' indices (row indices < 2^16 share
        // their top two bytes)
        uint32_t imin = 0xffffffffu, imax = 0u;
        for (int e = (int)lane; e < n; e += 32)
            if (pk[e] == vkey) {
                imin = min(imin, pi[e]);
                imax = max(imax, pi[e]);
            }
        imin = __reduce_min_sync(kFull, imin);
        imax = __reduce_max_sync(kFull, imax);  // (>= 2 distinct ties here: cnt > want >= 1)
        const int ifirst = __clz(imin ^ imax) >> 3;
        uint32_t ip = ifirst ? (imin & (0xffffffffu << (32 - 8 * ifirst))) : 0u;
#pragma unroll 1
        for (int pass = ifirst; pass < 4; ++pass) {
            const int shift = 24 - 8 * pass;
#pragma unroll
            for (int j = 0; j < 8; ++j) hist[j * 32 + lane] = 0u;
            __syncwarp();
            for (int e = (int)lane; e < n; e += 32) {
                if (pk[e] != vkey) continue;
                const uint32_t id = pi[e];
                const bool sel = (pass == ifirst) || ((id ^ ip) >> (shift + 8)) == 0u;
                if (sel) atomicAdd(&hist[hist_slot((id >> shift) & 255u)], 1u);
            }
            __syncwarp();
            const uint32_t d = hist_find(hist, lane, want, cnt);
            ip |= d << shift;
            __syncwarp();
        }
        idx = ip;
    }
    return ((unsigned long long)vkey << 32) | idx;
}

// In-place compaction of pool[0..n) to the pairs <= (tk, ti); returns the new count.
__device__ __noinline__ static int pool_compact(uint32_t* __restrict__ pk, uint32_t* __restrict__ pi, int n, uint32_t tk,
                                         uint32_t ti) {
    const uint32_t lane = lane_id();
    const uint32_t lt = lanemask_lt();
    int w = 0;
    for (int base = 0; base < n; base += 32) {
        const int e = base + (int)lane;
        uint32_t kk = 0, ii = 0;
        bool keep = false;
        if (e < n) {
            kk = pk[e];
            ii = pi[e];
            keep = !pair_lt(tk, ti, kk, ii);
        }
        const uint32_t bal = __ballot_sync(kFull, keep);
        __syncwarp();
        if (keep) {
            const int pos = w + __popc(bal & lt);
            pk[pos] = kk;
            pi[pos] = ii;
        }
        w += __popc(bal);
        __syncwarp();
    }
    return w;
}


// #{u : rk[u] < cand} for this lane, with four independent partial sums (the
// bisection steps below are latency-bound: a single add chain over NR compares
// would dominate them).
template <int NR>
__device__ __forceinline__ uint32_t count_lt(const uint32_t (&rk)[NR], uint32_t cand) {
    uint32_t c[4] = {0u, 0u, 0u, 0u};
#pragma unroll
    for (int u = 0; u < NR; ++u) c[u & 3] += (rk[u] < cand) ? 1u : 0u;
    return (c[0] + c[1]) + (c[2] + c[3]);
}

// Register-resident narrowing of one pool of n <= 32*NR pairs (global or shared
// memory): the pool is loaded once (NR pairs per lane), the want-th smallest
// pair is found by bisection on the key bits with warp-wide counts
// (__reduce_add_sync; no shared-memory histogram, hence no atomic contention
// when all keys share their top bits, e.g. distances), ties by a second
// bisection on the index, and the pool is compacted in place to the pairs
// <= that pair (exactly `want` of them).  Returns the pair; *n_out = want.
//
// slack > 0 (mid-stream narrowings): the bisection stops at the first candidate key c
// with want <= #{key < c} <= want + slack and keeps exactly those pairs; the returned
// bound (c - 1, 0x7ffffffe) -- "every index of key c - 1" -- still has >= want pairs at
// or below it.  A looser but valid threshold, found in a few steps instead of ~32 (the
// exact k-th is only needed at the end of a row).
template <int NR>
__device__ __noinline__ unsigned long long pool_narrow_regs(uint32_t* __restrict__ pk, uint32_t* __restrict__ pi,
                                                            int n, uint32_t want, int* n_out,
                                                            uint32_t* ties_out = nullptr, uint32_t slack = 0) {
    const uint32_t lane = lane_id();
    uint32_t rk[NR], ri[NR];
#pragma unroll
    for (int u = 0; u < NR; ++u) {
        const int x = u * 32 + (int)lane;
        rk[u] = (x < n) ? pk[x] : 0xffffffffu;  // generic loads: shared- or global-memory pools
        ri[u] = (x < n) ? pi[x] : 0xffffffffu;
    }
    // want-th smallest key: the largest v with #{key < v} < want (pads are
    // 0xffffffff: never below); bits above the highest bit where the smallest and
    // largest key differ are those of the smallest
    uint32_t kmin = 0xffffffffu, kmax = 0u;
#pragma unroll
    for (int u = 0; u < NR; ++u) {
        if (u * 32 + (int)lane < n) {
            kmin = min(kmin, rk[u]);
            kmax = max(kmax, rk[u]);
        }
    }
    kmin = __reduce_min_sync(kFull, kmin);
    kmax = __reduce_max_sync(kFull, kmax);
    const int top = (kmin == kmax) ? -1 : 31 - __clz(kmin ^ kmax);
    uint32_t vkey = (top < 0) ? kmin : (kmin & ~((2u << top) - 1u));
    uint32_t early = 0;  // (slack) candidate key whose "below" set fits [want, want + slack]
#pragma unroll 1
    for (int b = top; b >= 0; --b) {
        const uint32_t cand = vkey | (1u << b);
        const uint32_t c = __reduce_add_sync(kFull, count_lt<NR>(rk, cand));
        if (c < want) {
            vkey = cand;
        } else if (c <= want + slack && slack) {
            early = cand;
            break;
        }
    }
    uint32_t vidx;
    if (early) {  // keep every pair with key < early
        vkey = early - 1u;
        vidx = 0xffffffffu;
        if (ties_out) *ties_out = 0;
    } else {
        uint32_t less = 0, eq = 0, mx = 0;
#pragma unroll
        for (int u = 0; u < NR; ++u) {
            const bool valid = u * 32 + (int)lane < n;
            less += (rk[u] < vkey) ? 1u : 0u;
            const bool e = valid && rk[u] == vkey;
            eq += e ? 1u : 0u;
            mx = e ? max(mx, ri[u]) : mx;
        }
        less = __reduce_add_sync(kFull, less);
        eq = __reduce_add_sync(kFull, eq);
        if (ties_out) *ties_out = eq;
        const uint32_t need = want - less;  // ties of vkey to keep, in index order
        if (eq == need) {
            vidx = __reduce_max_sync(kFull, mx);
        } else {
            vidx = 0;
#pragma unroll 1
            for (int b = 31; b >= 0; --b) {
                const uint32_t cand = vidx | (1u << b);
                uint32_t c = 0;
#pragma unroll
                for (int u = 0; u < NR; ++u)
                    c += (u * 32 + (int)lane < n && rk[u] == vkey && ri[u] < cand) ? 1u : 0u;
                if (__reduce_add_sync(kFull, c) < need) vidx = cand;
            }
        }
    }
    // compaction in place: keep (key, idx) <= (vkey, vidx); every lane's loads above
    // precede any lane's stores below (the reductions already order them; the explicit
    // warp barrier makes that visible to racecheck)
    __syncwarp();
    const uint32_t lt = lanemask_lt();
    int w = 0;
#pragma unroll
    for (int u = 0; u < NR; ++u) {
        const bool keep = (u * 32 + (int)lane < n) && !pair_lt(vkey, vidx, rk[u], ri[u]);
        const uint32_t bal = __ballot_sync(kFull, keep);
        if (keep) {
            const int pos = w + __popc(bal & lt);
            pk[pos] = rk[u];
            pi[pos] = ri[u];
        }
        w += __popc(bal);
    }
    __syncwarp();
    *n_out = w;
    return ((unsigned long long)vkey << 32) | (early ? 0x7ffffffeu : vidx);
}

// Same as pool_narrow_regs for a pool of packed pairs (key << 32 | idx) in one
// u64 array; the key bisection starts below the common prefix of the pool's
// smallest and largest key.  GLOBAL: the pool is in global memory (L2 loads,
// __ldcg: other lanes wrote it); otherwise generic loads (shared memory).
// Compaction bound of a narrowing to the want-th pair T: T itself, or -- for pools of
// approximate keys (the fused k-NN's filter distances) -- every pair whose value is
// <= value(T) + band (band >= 0, rounded up; no finite bound keeps everything).
__device__ __forceinline__ unsigned long long band_bound(unsigned long long T, float band) {
    if (band < 0.f) return T;
    const uint32_t tk = (uint32_t)(T >> 32);
    if (tk >= 0xff800000u) return ~0ull;
    const float v = __fadd_ru(__uint_as_float(bits_of_key(tk)), band);
    if (!(v < __int_as_float(0x7f800000))) return ~0ull;
    const unsigned long long K = ((unsigned long long)key_of(v) << 32) | 0xffffffffull;
    return K > T ? K : T;
}

// band >= 0: keep the band above the want-th pair (band_bound); the want-th pair is returned.
template <int NR, bool GLOBAL = true>
// slack > 0: stop at the first candidate key c with want <= #{key < c} <= want + slack
// (as pool_narrow_regs) and return the key-level bound (c - 1, 0x7ffffffe).
__device__ __noinline__ unsigned long long pool_narrow64(unsigned long long* __restrict__ pool, int n, uint32_t want,
                                                         int* n_out, float band = -1.f, uint32_t slack = 0) {
    const uint32_t lane = lane_id();
    unsigned long long r[NR];
    uint32_t kmin = 0xffffffffu, kmax = 0u;
#pragma unroll
    for (int u = 0; u < NR; ++u) {
        const int x = u * 32 + (int)lane;
        r[u] = (x < n) ? (GLOBAL ? __ldcg(pool + x) : pool[x]) : 0xffffffffffffffffull;
        if (x < n) {
            kmin = min(kmin, (uint32_t)(r[u] >> 32));
            kmax = max(kmax, (uint32_t)(r[u] >> 32));
        }
    }
    kmin = __reduce_min_sync(kFull, kmin);
    kmax = __reduce_max_sync(kFull, kmax);
    // want-th smallest key: the largest v with #{key < v} < want; bits above the
    // highest bit where kmin and kmax differ are those of kmin
    const int top = (kmin == kmax) ? -1 : 31 - __clz(kmin ^ kmax);
    uint32_t vkey = (top < 0) ? kmin : (kmin & ~((2u << top) - 1u));
    uint32_t hk[NR];  // the key halves (pads: 0xffffffff, never below)
#pragma unroll
    for (int u = 0; u < NR; ++u) hk[u] = (uint32_t)(r[u] >> 32);
    uint32_t early = 0;
#pragma unroll 1
    for (int b = top; b >= 0; --b) {
        const uint32_t cand = vkey | (1u << b);
        const uint32_t c = __reduce_add_sync(kFull, count_lt<NR>(hk, cand));
        if (c < want) {
            vkey = cand;
        } else if (c <= want + slack && slack) {
            early = cand;
            break;
        }
    }
    uint32_t vidx;
    if (early) {
        vkey = early - 1u;
        vidx = 0x7ffffffeu;
    } else {
        uint32_t less = 0, eq = 0, mx = 0;
#pragma unroll
        for (int u = 0; u < NR; ++u) {
            const bool valid = u * 32 + (int)lane < n;
            const uint32_t kk = (uint32_t)(r[u] >> 32);
            less += (valid && kk < vkey) ? 1u : 0u;
            const bool e = valid && kk == vkey;
            eq += e ? 1u : 0u;
            mx = e ? max(mx, (uint32_t)r[u]) : mx;
        }
        less = __reduce_add_sync(kFull, less);
        eq = __reduce_add_sync(kFull, eq);
        const uint32_t need = want - less;
        if (eq == need) {
            vidx = __reduce_max_sync(kFull, mx);
        } else {
            vidx = 0;
#pragma unroll 1
            for (int b = 31; b >= 0; --b) {
                const uint32_t cand = vidx | (1u << b);
                uint32_t c = 0;
#pragma unroll
                for (int u = 0; u < NR; ++u)
                    c += (u * 32 + (int)lane < n && (uint32_t)(r[u] >> 32) == vkey && (uint32_t)r[u] < cand) ? 1u : 0u;
                if (__reduce_add_sync(kFull, c) < need) vidx = cand;
            }
        }
    }
    const unsigned long long T = ((unsigned long long)vkey << 32) | vidx;
    const unsigned long long K = band_bound(T, band);
    __syncwarp();  // all loads of the pool precede the in-place compaction
    const uint32_t lt = lanemask_lt();
    int w = 0;
#pragma unroll
    for (int u = 0; u < NR; ++u) {
        const bool keep = (u * 32 + (int)lane < n) && r[u] <= K;
        const uint32_t bal = __ballot_sync(kFull, keep);
        if (keep) pool[w + __popc(bal & lt)] = r[u];
        w += __popc(bal);
    }
    __syncwarp();
    *n_out = w;
    return T;
}

// Visit pool[0..n) in batches of 8 loads per lane (8 L2 requests in flight
// before any use: the passes below are latency-bound otherwise, since the
// compiler cannot hoist a global load above a shared-memory atomic of the
// previous element); f(v) on every valid entry.
template <bool GLOBAL = true, typename F>
__device__ __forceinline__ void pool_scan64(const unsigned long long* __restrict__ pool, int n, uint32_t lane, F f) {
#pragma unroll 1
    for (int base = 0; base < n; base += 256) {
        unsigned long long v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const int e = base + j * 32 + (int)lane;
            v[j] = (e < n) ? (GLOBAL ? __ldcg(pool + e) : pool[e]) : 0ull;
        }
#pragma unroll
        for (int j = 0; j < 8; ++j)
            if (base + j * 32 + (int)lane < n) f(v[j]);
    }
}

// Radix select for large packed-pair pools (key << 32 | idx, any memory): the
// want-th smallest pair by MSD 8-bit digits of the key, starting below the
// common prefix of the pool's smallest and largest key (distances share their
// top bits), then of the index for ties; shared-memory histogram `hist` (256 u32,
// transposed layout).  The pool is then compacted in place to the pairs <= it.
// slack > 0: stop after the first key digit whose bucket, with everything below it,
// holds at most want + slack pairs; the bound is then (bucket's last key, 0x7ffffffe).
// (GLOBAL = false: a shared-memory pool -- generic loads instead of ld.global.cg)
template <bool GLOBAL = true>
__device__ __noinline__ unsigned long long pool_select64(unsigned long long* __restrict__ pool, int n,
                                                               uint32_t want, uint32_t* __restrict__ hist,
                                                               int* n_out, float band = -1.f, uint32_t slack = 0) {
    const uint32_t want0 = want;
    bool early = false;
    const uint32_t lane = lane_id();
    uint32_t kmin = 0xffffffffu, kmax = 0u;
    pool_scan64<GLOBAL>(pool, n, lane, [&](unsigned long long v) {
        const uint32_t kk = (uint32_t)(v >> 32);
        kmin = min(kmin, kk);
        kmax = max(kmax, kk);
    });
    kmin = __reduce_min_sync(kFull, kmin);
    kmax = __reduce_max_sync(kFull, kmax);
    int hi = (kmin == kmax) ? -1 : 31 - __clz(kmin ^ kmax);
    uint32_t prefix = (hi < 0) ? kmin : (kmin & ~((2u << hi) - 1u));
    uint32_t cnt = (uint32_t)n;  // entries matching the resolved prefix (all, initially)
    // key digits
    while (hi >= 0) {
        const int lo = hi >= 7 ? hi - 7 : 0;
        const uint32_t dmask = (2u << (hi - lo)) - 1u;
#pragma unroll
        for (int j = 0; j < 8; ++j) hist[j * 32 + lane] = 0u;
        __syncwarp();
        pool_scan64<GLOBAL>(pool, n, lane, [&](unsigned long long v) {
            const uint32_t kk = (uint32_t)(v >> 32);
            const bool sel = (hi == 31) || ((kk ^ prefix) >> (hi + 1)) == 0u;
            if (sel) atomicAdd(&hist[hist_slot((kk >> lo) & dmask)], 1u);
        });
        __syncwarp();
        const uint32_t d = hist_find(hist, lane, want, cnt);
        prefix |= d << lo;
        __syncwarp();
        if (slack && (want0 - want) + cnt <= want0 + slack) {  // take the whole bucket
            prefix |= (1u << lo) - 1u;
            early = true;
            break;
        }
        hi = lo - 1;
    }
    const uint32_t vkey = prefix;
    uint32_t vidx;
    if (early) {
        vidx = 0x7ffffffeu;
    } else if (cnt == want) {
        uint32_t m = 0;
        pool_scan64<GLOBAL>(pool, n, lane, [&](unsigned long long v) {
            if ((uint32_t)(v >> 32) == vkey) m = max(m, (uint32_t)v);
        });
        vidx = __reduce_max_sync(kFull, m);
    } else {
        uint32_t ip = 0;
#pragma unroll 1
        for (int pass = 0; pass < 4; ++pass) {
            const int shift = 24 - 8 * pass;
#pragma unroll
            for (int j = 0; j < 8; ++j) hist[j * 32 + lane] = 0u;
            __syncwarp();
            pool_scan64<GLOBAL>(pool, n, lane, [&](unsigned long long v) {
                if ((uint32_t)(v >> 32) != vkey) return;
                const uint32_t id = (uint32_t)v;
                const bool sel = (pass == 0) || ((id ^ ip) >> (shift + 8)) == 0u;
                if (sel) atomicAdd(&hist[hist_slot((id >> shift) & 255u)], 1u);
            });
            __syncwarp();
            const uint32_t d = hist_find(hist, lane, want, cnt);
            ip |= d << shift;
            __syncwarp();
        }
        vidx = ip;
    }
    const unsigned long long T = ((unsigned long long)vkey << 32) | vidx;
    const unsigned long long K = band_bound(T, band);
    // in-place compaction, 8 slabs of 32 per batch: every read of a batch precedes its
    // writes, and writes never pass the batch's first slab (w <= base)
    const uint32_t lt = lanemask_lt();
    int w = 0;
#pragma unroll 1
    for (int base = 0; base < n; base += 256) {
        unsigned long long v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const int e = base + j * 32 + (int)lane;
            v[j] = (e < n) ? (GLOBAL ? __ldcg(pool + e) : pool[e]) : ~0ull;
        }
        __syncwarp();
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const bool keep = base + j * 32 + (int)lane < n && v[j] <= K;
            const uint32_t bal = __ballot_sync(kFull, keep);
            if (keep) pool[w + __popc(bal & lt)] = v[j];
            w += __popc(bal);
        }
    }
    __syncwarp();
    *n_out = w;
    return T;
}

}  // namespace ksel
