// paper_variants.cu -- the paper's own per-thread selection designs on B200
// (ablation kernels, not the hot path).
//
// One thread per query, the distance matrix stored query-
// contiguous, dist_t[N][Q] (element (q, j) at j*Q + q), so that a warp's 32
// threads read 128 consecutive bytes per step -- the coalescing the paper's HP
// construction relies on (L225; reading R10).  Per-thread queues, buffers and
// HP levels live in a global workspace, laid out [position][Q] (coalesced for
// warp-synchronous positions), as the paper's per-thread structures must have
// (8192 threads x 1024 pairs do not fit 48 KB of shared memory, L243).
//
// Variants (any combination):
//   queue  KSEL_PQ_INSERT  sorted array, max at head, O(k) insertion (L17, L37, Fig. 1a)
//          KSEL_PQ_HEAP    max-heap, O(log k) (L17, L37)
//          KSEL_PQ_MERGE   Merge Queue, Alg. 2 (L39-L41): levels m, m, 2m, ..., k/2,
//                          each sorted decreasing; insertion sort into level 1 and
//                          lazy merges of the sorted prefix with the next level
//                          (Reverse Bitonic Merge, Fig. 2) while some deeper
//                          head is above the first (readings R11, R11b);
//          KSEL_PQ_MERGE_ALIGNED  the same, merges taken by the whole warp when any
//                          lane needs one (the intra-warp flag, L183; here a vote)
//   buffer KSEL_PB_NONE | KSEL_PB_BUFFER (Alg. 3, per-thread flush when its own buffer
//          is full) | KSEL_PB_FULL (the warp flushes when any buffer is full, L185) |
//          KSEL_PB_FULL_SORTED (+ Local Sort of the buffer before the flush, L187);
//          the last partial buffer is flushed (reading R14)
//   hp_G   0 = off, else Hierarchical Partition with group size G (Alg. 4, L221-
//          L231): bottom-up levels of (min value, index of its first minimum) until
//          <= k entries, then top-down: the top level's entries are the first
//          candidates; at each level the children [iG, (i+1)G) of the k
//          lexicographically smallest entries are the next candidates (reading R13).
// Every variant keeps the k lexicographically smallest (value, index) pairs
// (readings R1-R5: order keys, lower index first on equal values), so the
// result is bit-identical to ksel_select; the output is sorted ascending (R2).
#include <cstdint>

#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_common.cuh"
#include "ksel_internal.h"

namespace ksel {

constexpr int PV_THREADS = 128;
constexpr int PV_MAX_LEVELS = 40;

struct PaperArgs {
    const float* dist_t;
    int64_t Q, N;
    int k;        // requested k
    int kq;       // queue capacity (k, or for the Merge Queue m * 2^j >= k)
    int m;        // Merge Queue level-1 size
    int bsize;    // per-thread candidate buffer
    int G;        // HP group size (0: off)
    int nlev;     // HP levels above the row
    int64_t lev_off[PV_MAX_LEVELS];   // offset (pairs per query) of level l (1-based) in lk/li
    int64_t lev_size[PV_MAX_LEVELS];  // entries of level l (lev_size[0] = N)
    int64_t gpow[PV_MAX_LEVELS];      // G^l
    uint32_t *qk, *qi;  // queue    [kq][Q]
    uint32_t *bk, *bi;  // buffer   [bsize][Q]
    uint32_t *lk, *li;  // HP levels [sum sizes][Q]
    uint32_t *tk, *ti;  // HP: previous level's selection [kq][Q]
    float* ov;
    int32_t* oi;
};

__device__ __forceinline__ bool pgt(uint32_t ka, uint32_t ia, uint32_t kb, uint32_t ib) {
    return pair_lt(kb, ib, ka, ia);
}

template <int QUEUE, int BUF>
__global__ void __launch_bounds__(PV_THREADS) ksel_paper_kernel(const PaperArgs A) {
    const int64_t q = (int64_t)blockIdx.x * PV_THREADS + threadIdx.x;
    const bool active = q < A.Q;
    const int64_t Q = A.Q;
    const int64_t qq = active ? q : 0;
    auto QK = [&](int64_t p) -> uint32_t& { return A.qk[p * Q + qq]; };
    auto QI = [&](int64_t p) -> uint32_t& { return A.qi[p * Q + qq]; };
    auto BK = [&](int64_t p) -> uint32_t& { return A.bk[p * Q + qq]; };
    auto BI = [&](int64_t p) -> uint32_t& { return A.bi[p * Q + qq]; };
    const int kq = A.kq;
    constexpr bool ALIGNED = (QUEUE == KSEL_PQ_MERGE_ALIGNED);

    auto reset_queue = [&]() {
        if (active)
            for (int p = 0; p < kq; ++p) { QK(p) = kSentKey; QI(p) = kSentIdx; }
    };
    // two decreasing runs [0, L) and [L, 2L) -> decreasing [0, 2L): flip + clean (Fig. 2)
    auto merge_desc = [&](int L) {
        for (int i = 0; i < L; ++i) {
            const int j = 2 * L - 1 - i;
            const uint32_t ka = QK(i), ia = QI(i), kb = QK(j), ib = QI(j);
            if (pair_lt(ka, ia, kb, ib)) { QK(i) = kb; QI(i) = ib; QK(j) = ka; QI(j) = ia; }
        }
        for (int s = L >> 1; s > 0; s >>= 1)
            for (int h = 0; h < 2 * L; h += L)
                for (int i = h; i < h + L; ++i)
                    if ((i & s) == 0) {
                        const int j = i + s;
                        const uint32_t ka = QK(i), ia = QI(i), kb = QK(j), ib = QI(j);
                        if (pair_lt(ka, ia, kb, ib)) { QK(i) = kb; QI(i) = ib; QK(j) = ka; QI(j) = ia; }
                    }
    };
    // insert (key, idx), known to be below the head (the queue's maximum)
    auto insert_pred = [&](bool doit, uint32_t key, uint32_t idx) {
        if (QUEUE == KSEL_PQ_INSERT) {
            if (doit) {
                int p = 0;
                while (p + 1 < kq && pgt(QK(p + 1), QI(p + 1), key, idx)) {
                    QK(p) = QK(p + 1); QI(p) = QI(p + 1);
                    ++p;
                }
                QK(p) = key; QI(p) = idx;
            }
        } else if (QUEUE == KSEL_PQ_HEAP) {
            if (doit) {
                int p = 0;
                while (true) {
                    const int l = 2 * p + 1;
                    if (l >= kq) break;
                    int c = l;
                    if (l + 1 < kq && pgt(QK(l + 1), QI(l + 1), QK(l), QI(l))) c = l + 1;
                    if (!pgt(QK(c), QI(c), key, idx)) break;
                    QK(p) = QK(c); QI(p) = QI(c);
                    p = c;
                }
                QK(p) = key; QI(p) = idx;
            }
        } else {  // Merge Queue: insertion sort into level 1 (replacing the head) ...
            if (doit) {
                int p = 0;
                while (p + 1 < A.m && pgt(QK(p + 1), QI(p + 1), key, idx)) {
                    QK(p) = QK(p + 1); QI(p) = QI(p + 1);
                    ++p;
                }
                QK(p) = key; QI(p) = idx;
            }
            // ... then lazy merges: while some deeper level's head is above the head, merge
            // the sorted prefix [0, L) with the next level (prefix sizes m, 2m, 4m, ...).
            // Comparing only consecutive heads (Alg. 2 as printed) is not enough: after a
            // merge the second level's new head can sit below the third level's, and a
            // later insertion then leaves a larger head deeper in the queue (reading R11b,
            // found by simulation; this form keeps the exact k smallest in every stream).
            for (int L = A.m; L < kq; L <<= 1) {
                bool need = false;
                if (doit)
                    for (int H = L; H < kq; H <<= 1) need |= pair_lt(QK(0), QI(0), QK(H), QI(H));
                if (ALIGNED) need = __any_sync(kFull, need);
                if (!need) break;
                if (active) merge_desc(L);  // (lanes past Q have no queue of their own)
            }
        }
    };

    int c = 0;  // buffered candidates
    auto flush = [&]() {
        if (BUF == KSEL_PB_FULL_SORTED) {  // Local Sort (ascending) before inserting
            for (int i = 1; i < c; ++i) {
                const uint32_t kk = BK(i), ii = BI(i);
                int j = i - 1;
                while (j >= 0 && pgt(BK(j), BI(j), kk, ii)) { BK(j + 1) = BK(j); BI(j + 1) = BI(j); --j; }
                BK(j + 1) = kk; BI(j + 1) = ii;
            }
        }
        const int cmax = ALIGNED ? __reduce_max_sync(kFull, (uint32_t)c) : c;
        for (int i = 0; i < cmax; ++i) {
            const bool has = i < c;
            const uint32_t kk = has ? BK(i) : 0u, ii = has ? BI(i) : 0u;
            const bool doit = has && pair_lt(kk, ii, QK(0), QI(0));  // re-tested against the current head
            insert_pred(doit, kk, ii);
        }
        c = 0;
    };
    // one candidate of a stream (every lane calls this the same number of times)
    auto consume = [&](bool valid, uint32_t key, uint32_t idx) {
        const bool admit = valid && pair_lt(key, idx, QK(0), QI(0));
        if (BUF == KSEL_PB_NONE) {
            insert_pred(admit, key, idx);
            return;
        }
        if (admit) { BK(c) = key; BI(c) = idx; ++c; }
        const bool full = c == A.bsize;
        if (BUF == KSEL_PB_BUFFER) {
            if (!ALIGNED) {
                if (full) flush();
            } else if (__any_sync(kFull, full)) {
                flush();  // merges must stay warp-uniform
            }
        } else if (__any_sync(kFull, full)) {  // the intra-warp "buffer full" flag (L185)
            flush();
        }
    };
    auto row_key = [&](int64_t j) { return key_of(A.dist_t[j * Q + qq]); };

    reset_queue();
    if (A.G == 0 || A.nlev == 0) {
        for (int64_t j = 0; j < A.N; ++j) consume(active, active ? row_key(j) : 0u, (uint32_t)j);
        flush();
    } else {
        const int G = A.G;
        // ---- HP bottom-up (Alg. 4): level l entry p = the lexicographic minimum of its
        // G children (value key, index of the first minimum) ----
        if (active) {
            for (int l = 1; l <= A.nlev; ++l) {
                const int64_t n = A.lev_size[l], np = A.lev_size[l - 1];
                for (int64_t p = 0; p < n; ++p) {
                    uint32_t bk = kSentKey, bi = kSentIdx;
                    for (int64_t ch = p * G; ch < p * G + G && ch < np; ++ch) {
                        uint32_t ck, ci;
                        if (l == 1) { ck = row_key(ch); ci = (uint32_t)ch; }
                        else { ck = A.lk[(A.lev_off[l - 1] + ch) * Q + qq]; ci = A.li[(A.lev_off[l - 1] + ch) * Q + qq]; }
                        if (pair_lt(ck, ci, bk, bi)) { bk = ck; bi = ci; }
                    }
                    A.lk[(A.lev_off[l] + p) * Q + qq] = bk;
                    A.li[(A.lev_off[l] + p) * Q + qq] = bi;
                }
            }
        }
        // ---- HP top-down: the top level's entries, then the children of each level's selection ----
        const int top = A.nlev;
        for (int64_t p = 0; p < A.lev_size[top]; ++p)
            consume(active, active ? A.lk[(A.lev_off[top] + p) * Q + qq] : 0u,
                    active ? A.li[(A.lev_off[top] + p) * Q + qq] : 0u);
        flush();
        for (int l = top; l >= 1; --l) {
            if (active)
                for (int p = 0; p < kq; ++p) { A.tk[(int64_t)p * Q + qq] = QK(p); A.ti[(int64_t)p * Q + qq] = QI(p); }
            reset_queue();
            const int64_t nc = A.lev_size[l - 1];
            for (int p = 0; p < kq; ++p) {
                const uint32_t ek = active ? A.tk[(int64_t)p * Q + qq] : kSentKey;
                const uint32_t ei = active ? A.ti[(int64_t)p * Q + qq] : kSentIdx;
                const bool real = !(ek == kSentKey && ei == kSentIdx);
                const int64_t P = real ? (int64_t)ei / A.gpow[l] : 0;  // its position at level l
                for (int g = 0; g < G; ++g) {
                    const int64_t ch = P * G + g;
                    const bool v = active && real && ch < nc;
                    uint32_t ck = 0, ci = 0;
                    if (v) {
                        if (l == 1) { ck = row_key(ch); ci = (uint32_t)ch; }
                        else { ck = A.lk[(A.lev_off[l - 1] + ch) * Q + qq]; ci = A.li[(A.lev_off[l - 1] + ch) * Q + qq]; }
                    }
                    consume(v, ck, ci);
                }
            }
            flush();
        }
    }
    if (!active) return;

    // ---- emit: the queue's k smallest, ascending (heap sort; the insertion queue is
    // already sorted decreasing) ----
    if (QUEUE != KSEL_PQ_INSERT) {
        // build a max-heap (the Merge Queue's levels are not one), then pop to the back
        for (int s = kq / 2 - 1; s >= 0; --s) {
            int p = s;
            const uint32_t key = QK(p), idx = QI(p);
            while (true) {
                const int l = 2 * p + 1;
                if (l >= kq) break;
                int ch = l;
                if (l + 1 < kq && pgt(QK(l + 1), QI(l + 1), QK(l), QI(l))) ch = l + 1;
                if (!pgt(QK(ch), QI(ch), key, idx)) break;
                QK(p) = QK(ch); QI(p) = QI(ch);
                p = ch;
            }
            QK(p) = key; QI(p) = idx;
        }
        for (int end = kq - 1; end > 0; --end) {
            const uint32_t key = QK(end), idx = QI(end);
            QK(end) = QK(0); QI(end) = QI(0);
            int p = 0;
            while (true) {
                const int l = 2 * p + 1;
                if (l >= end) break;
                int ch = l;
                if (l + 1 < end && pgt(QK(l + 1), QI(l + 1), QK(l), QI(l))) ch = l + 1;
                if (!pgt(QK(ch), QI(ch), key, idx)) break;
                QK(p) = QK(ch); QI(p) = QI(ch);
                p = ch;
            }
            QK(p) = key; QI(p) = idx;
        }
    }
    float* ov = A.ov + q * (int64_t)A.k;
    int32_t* oi = A.oi + q * (int64_t)A.k;
    for (int e = 0; e < A.k; ++e) {
        const int p = (QUEUE == KSEL_PQ_INSERT) ? kq - 1 - e : e;  // ascending position
        const uint32_t kk = QK(p), ii = QI(p);
        const uint32_t bits = key_needs_regather(kk) ? __float_as_uint(A.dist_t[(int64_t)ii * Q + q]) : bits_of_key(kk);
        ov[e] = __uint_as_float(bits);
        oi[e] = (int32_t)ii;
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
static int paper_plan(int64_t Q, int64_t N, int k, int queue, int buf, int G, int m, int bsize, PaperArgs* A,
                      size_t* bytes) {
    if (Q < 1 || N < 1 || N > 0x7fffffffLL || k < 1 || k > N) return KSEL_ERR_INVALID_ARG;
    if (k > KSEL_MAX_K) return KSEL_ERR_UNSUPPORTED;
    if (queue < KSEL_PQ_INSERT || queue > KSEL_PQ_MERGE_ALIGNED || buf < KSEL_PB_NONE || buf > KSEL_PB_FULL_SORTED)
        return KSEL_ERR_INVALID_ARG;
    if (G != 0 && (G < 2 || G > 64)) return KSEL_ERR_INVALID_ARG;
    if (m < 1 || m > 1024 || (m & (m - 1)) || bsize < 1 || bsize > 1024) return KSEL_ERR_INVALID_ARG;
    PaperArgs a{};
    a.Q = Q;
    a.N = N;
    a.k = k;
    a.m = m;
    a.bsize = bsize;
    a.G = G;
    a.kq = k;
    if (queue == KSEL_PQ_MERGE || queue == KSEL_PQ_MERGE_ALIGNED) {
        int kq = m;
        while (kq < k) kq <<= 1;
        if (kq < 2 * m) kq = 2 * m;  // at least levels 1 and 2 (L41)
        if (kq > 2 * KSEL_MAX_K) return KSEL_ERR_UNSUPPORTED;
        a.kq = kq;
    }
    a.lev_size[0] = N;
    a.gpow[0] = 1;
    int64_t tot = 0;
    if (G) {
        int l = 0;
        while (a.lev_size[l] > a.kq) {  // Alg. 4: build until the top level fits the queue
            if (l + 1 >= PV_MAX_LEVELS) return KSEL_ERR_UNSUPPORTED;
            a.lev_size[l + 1] = (a.lev_size[l] + G - 1) / G;
            a.gpow[l + 1] = a.gpow[l] * G;
            a.lev_off[l + 1] = tot;
            tot += a.lev_size[l + 1];
            ++l;
        }
        a.nlev = l;
    }
    const size_t q4 = (size_t)Q * 4u;
    auto al = [](size_t x) { return (x + 255u) & ~(size_t)255u; };
    size_t off = 0;
    const size_t o_qk = off; off += al((size_t)a.kq * q4);
    const size_t o_qi = off; off += al((size_t)a.kq * q4);
    const size_t o_bk = off; off += al((size_t)bsize * q4);
    const size_t o_bi = off; off += al((size_t)bsize * q4);
    const size_t o_lk = off; off += al((size_t)(tot ? tot : 1) * q4);
    const size_t o_li = off; off += al((size_t)(tot ? tot : 1) * q4);
    const size_t o_tk = off; off += al((size_t)a.kq * q4);
    const size_t o_ti = off; off += al((size_t)a.kq * q4);
    *bytes = off;
    if (A) {
        uint8_t* w = nullptr;  // offsets only; the caller adds the base
        a.qk = reinterpret_cast<uint32_t*>(w + o_qk);
        a.qi = reinterpret_cast<uint32_t*>(w + o_qi);
        a.bk = reinterpret_cast<uint32_t*>(w + o_bk);
        a.bi = reinterpret_cast<uint32_t*>(w + o_bi);
        a.lk = reinterpret_cast<uint32_t*>(w + o_lk);
        a.li = reinterpret_cast<uint32_t*>(w + o_li);
        a.tk = reinterpret_cast<uint32_t*>(w + o_tk);
        a.ti = reinterpret_cast<uint32_t*>(w + o_ti);
        *A = a;
    }
    return KSEL_OK;
}

template <int QUEUE>
static cudaError_t launch_paper_q(int buf, const PaperArgs& a, cudaStream_t stream) {
    const unsigned grid = (unsigned)((a.Q + PV_THREADS - 1) / PV_THREADS);
    switch (buf) {
        case KSEL_PB_NONE: ksel_paper_kernel<QUEUE, KSEL_PB_NONE><<<grid, PV_THREADS, 0, stream>>>(a); break;
        case KSEL_PB_BUFFER: ksel_paper_kernel<QUEUE, KSEL_PB_BUFFER><<<grid, PV_THREADS, 0, stream>>>(a); break;
        case KSEL_PB_FULL: ksel_paper_kernel<QUEUE, KSEL_PB_FULL><<<grid, PV_THREADS, 0, stream>>>(a); break;
        default: ksel_paper_kernel<QUEUE, KSEL_PB_FULL_SORTED><<<grid, PV_THREADS, 0, stream>>>(a); break;
    }
    note_launch();
    return cudaGetLastError();
}

}  // namespace ksel

using namespace ksel;

extern "C" {

size_t ksel_select_paper_workspace(int64_t Q, int64_t N, int k, int queue, int buffer, int hp_G, int m, int bsize) {
    size_t bytes = 0;
    return paper_plan(Q, N, k, queue, buffer, hp_G, m, bsize, nullptr, &bytes) == KSEL_OK ? bytes : 0;
}

int ksel_select_paper(const float* dist_t, int64_t Q, int64_t N, int k, int queue, int buffer, int hp_G, int m,
                      int bsize, float* out_val, int32_t* out_idx, void* d_work, size_t work_bytes, void* stream) {
    if (!dist_t || !out_val || !out_idx || !d_work) return KSEL_ERR_INVALID_ARG;
    PaperArgs a;
    size_t bytes = 0;
    int st = paper_plan(Q, N, k, queue, buffer, hp_G, m, bsize, &a, &bytes);
    if (st) return st;
    if (work_bytes < bytes) return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    uint8_t* w = static_cast<uint8_t*>(d_work);
    auto rebase = [&](uint32_t*& p) { p = reinterpret_cast<uint32_t*>(w + reinterpret_cast<uintptr_t>(p)); };
    rebase(a.qk); rebase(a.qi); rebase(a.bk); rebase(a.bi); rebase(a.lk); rebase(a.li); rebase(a.tk); rebase(a.ti);
    a.dist_t = dist_t;
    a.ov = out_val;
    a.oi = out_idx;
    const cudaStream_t s = (cudaStream_t)stream;
    const int slot = timing_begin(s);
    cudaError_t e;
    switch (queue) {
        case KSEL_PQ_INSERT: e = launch_paper_q<KSEL_PQ_INSERT>(buffer, a, s); break;
        case KSEL_PQ_HEAP: e = launch_paper_q<KSEL_PQ_HEAP>(buffer, a, s); break;
        case KSEL_PQ_MERGE: e = launch_paper_q<KSEL_PQ_MERGE>(buffer, a, s); break;
        default: e = launch_paper_q<KSEL_PQ_MERGE_ALIGNED>(buffer, a, s); break;
    }
    timing_end(slot, s);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

}  // extern "C"
