// api.cu -- the C ABI of libksel.so (declared in include/ksel.h).
//
// Host-side argument validation, device-property cache, launch dispatch and
// the host-buffer (end-to-end) pipeline.  No torch types, no allocation on the
// device paths, no stream synchronisation except in ksel_select_host.
#include <atomic>
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_internal.h"

namespace ksel {

static std::atomic<int64_t> g_launches{0};
void note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

cudaError_t ensure_smem_attr(const void* func, int bytes) {
    static std::mutex mu;
    struct Entry {
        const void* f;
        int dev;
        int bytes;
    };
    static Entry done[256];
    static int ndone = 0;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lock(mu);
    for (int i = 0; i < ndone; ++i)
        if (done[i].f == func && done[i].dev == dev && done[i].bytes >= bytes) return cudaSuccess;
    e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess && ndone < 256) done[ndone++] = Entry{func, dev, bytes};
    return e;
}

// ---- dominant-kernel timing ------------------------------------------------
static std::mutex g_tm_mu;
static bool g_tm_on = false;
struct TimedLaunch {
    cudaEvent_t a, b;
};
static TimedLaunch g_tm[4096];
static int g_tm_n = 0;

int timing_begin(cudaStream_t stream) {
    std::lock_guard<std::mutex> lock(g_tm_mu);
    if (!g_tm_on || g_tm_n >= 4096) return -1;
    TimedLaunch& t = g_tm[g_tm_n];
    if (cudaEventCreate(&t.a) != cudaSuccess) return -1;
    if (cudaEventCreate(&t.b) != cudaSuccess) { cudaEventDestroy(t.a); return -1; }
    cudaEventRecord(t.a, stream);
    return g_tm_n++;
}

void timing_end(int slot, cudaStream_t stream) {
    if (slot < 0) return;
    std::lock_guard<std::mutex> lock(g_tm_mu);
    cudaEventRecord(g_tm[slot].b, stream);
}

int env_int(const char* name, int dflt) {
    const char* e = std::getenv(name);
    return (e && e[0]) ? std::atoi(e) : dflt;
}

int chunk_order_mode() {
    // bits 0-1: chunk visit order (KSEL_ORDER, default 3); bit 2: loose admission
    // experiment (KSEL_LOOSE=1).  Experiments only; the defaults are the product.
    static const int mode = [] {
        const char* e = std::getenv("KSEL_ORDER");
        int m = (e && e[0] >= '0' && e[0] <= '3') ? e[0] - '0' : 3;
        const char* l = std::getenv("KSEL_LOOSE");
        if (l && l[0] == '1') m |= 4;
        // bit 6: no speculative starting bound (KSEL_SPEC=0; result-preserving)
        const char* sp = std::getenv("KSEL_SPEC");
        if (sp && sp[0] == '0') m |= 64;
#ifdef KSEL_EXPERIMENTS
        // phase-cost experiments of the pool kernel (results are wrong): bit 3 = no exact
        // admission path, bit 4 = no final select/sort/merge, bit 5 = no starting bound
        m |= env_int("KSEL_POOL_SKIP", 0) & (8 | 16 | 32);
#endif
        return m;
    }();
    return mode;
}

static std::mutex g_dev_mu;
static DevInfo g_dev[64];
static bool g_dev_ok[64];

int current_device_info(DevInfo* out) {
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return KSEL_ERR_NO_DEVICE;
    std::lock_guard<std::mutex> lock(g_dev_mu);
    if (!g_dev_ok[dev]) {
        cudaDeviceProp p;
        if (cudaGetDeviceProperties(&p, dev) != cudaSuccess) return KSEL_ERR_CUDA;
        g_dev[dev].dev = dev;
        g_dev[dev].sms = p.multiProcessorCount;
        g_dev[dev].major = p.major;
        g_dev[dev].minor = p.minor;
        g_dev_ok[dev] = true;
    }
    *out = g_dev[dev];
    if (out->major != 10) return KSEL_ERR_NO_DEVICE;  // built for sm_100a only
    return KSEL_OK;
}

static size_t al256(size_t x) { return (x + 255u) & ~(size_t)255u; }

static bool overlaps(const void* a, size_t na, const void* b, size_t nb) {
    const uintptr_t x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
    return x < y + nb && y < x + na;
}

static int check_select_args(const float* dist, int64_t Q, int64_t N, int k, const float* ov, const int32_t* oi) {
    if (!dist || !ov || !oi) return KSEL_ERR_INVALID_ARG;
    if (Q < 1 || N < 1 || N > 0x7fffffffLL || k < 1 || k > N) return KSEL_ERR_INVALID_ARG;
    if ((reinterpret_cast<uintptr_t>(dist) & 3u) || (reinterpret_cast<uintptr_t>(ov) & 3u) ||
        (reinterpret_cast<uintptr_t>(oi) & 3u))
        return KSEL_ERR_INVALID_ARG;
    if (k > KSEL_MAX_K) return KSEL_ERR_UNSUPPORTED;
    return KSEL_OK;
}

}  // namespace ksel

using namespace ksel;

extern "C" {

int ksel_version(void) { return 100; }  // 0.1.0

int64_t ksel_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

int ksel_timing_enable(int on) {
    std::lock_guard<std::mutex> lock(g_tm_mu);
    g_tm_on = on != 0;
    return KSEL_OK;
}

int ksel_timing_collect(double* total_ms, int64_t* launches) {
    if (!total_ms || !launches) return KSEL_ERR_INVALID_ARG;
    std::lock_guard<std::mutex> lock(g_tm_mu);
    double tot = 0.0;
    int st = KSEL_OK;
    for (int i = 0; i < g_tm_n; ++i) {
        float ms = 0.f;
        if (cudaEventSynchronize(g_tm[i].b) != cudaSuccess ||
            cudaEventElapsedTime(&ms, g_tm[i].a, g_tm[i].b) != cudaSuccess)
            st = KSEL_ERR_CUDA;
        tot += ms;
        cudaEventDestroy(g_tm[i].a);
        cudaEventDestroy(g_tm[i].b);
    }
    *total_ms = tot;
    *launches = g_tm_n;
    g_tm_n = 0;
    return st;
}

const char* ksel_strerror(int status) {
    switch (status) {
        case KSEL_OK: return "success";
        case KSEL_ERR_INVALID_ARG: return "invalid argument";
        case KSEL_ERR_UNSUPPORTED: return "unsupported configuration (k > 1024?)";
        case KSEL_ERR_CUDA: return "CUDA runtime error";
        case KSEL_ERR_NO_DEVICE: return "no sm_100 (B200) device is current";
        case KSEL_ERR_TIMEOUT: return "a device-side flag wait timed out (exchange results invalid)";
        default: return "unknown ksel status";
    }
}

int ksel_select_config(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx, int algo,
                       int warps_per_row, void* stream) {
    int st = check_select_args(dist, Q, N, k, out_val, out_idx);
    if (st) return st;
    if (algo < KSEL_ALGO_AUTO || algo > KSEL_ALGO_HIST) return KSEL_ERR_INVALID_ARG;
    if (algo == KSEL_ALGO_RADIX && !radix_supported(N, k)) return KSEL_ERR_UNSUPPORTED;
    if (algo == KSEL_ALGO_HIST && !hist_supported(N, k)) return KSEL_ERR_UNSUPPORTED;  // (experiments build only)
    if (warps_per_row != 0 && warps_per_row != 1 && warps_per_row != 2 && warps_per_row != 4 && warps_per_row != 8)
        return KSEL_ERR_INVALID_ARG;
    const size_t in_bytes = (size_t)Q * (size_t)N * 4u, out_bytes = (size_t)Q * (size_t)k * 4u;
    if (overlaps(dist, in_bytes, out_val, out_bytes) || overlaps(dist, in_bytes, out_idx, out_bytes) ||
        overlaps(out_val, out_bytes, out_idx, out_bytes))
        return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    if (algo == KSEL_ALGO_AUTO) algo = KSEL_ALGO_POOL;
    const int slot = timing_begin((cudaStream_t)stream);
    cudaError_t e;
    if (algo == KSEL_ALGO_RADIX) {
        e = launch_select_radix(dist, Q, N, k, out_val, out_idx, (cudaStream_t)stream);
    } else if (algo == KSEL_ALGO_HIST) {
        e = launch_select_hist(dist, Q, N, k, out_val, out_idx, di.sms, (cudaStream_t)stream);
    } else if (algo == KSEL_ALGO_QUEUE) {
        const int wpr = warps_per_row ? warps_per_row : stream_warps_per_row(Q, N, di.sms);
        e = launch_select_stream(dist, Q, N, k, out_val, out_idx, wpr, (cudaStream_t)stream);
    } else {
        const int shape = pool_launch_shape(Q, N, k, di.sms, warps_per_row);
        e = launch_select_pool(dist, Q, N, k, out_val, out_idx, shape, (cudaStream_t)stream);
    }
    timing_end(slot, (cudaStream_t)stream);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_select(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx,
                void* stream) {
    return ksel_select_config(dist, Q, N, k, out_val, out_idx, KSEL_ALGO_AUTO, 0, stream);
}

// ---------------------------------------------------------------------------
// split rows: few rows cannot fill the GPU with row parallelism
// (a row lives in one CTA of <= 8 warps), so each row is cut into S segments and
// every segment selects its own top-k (the pool kernel on Q*S virtual rows,
// row-global indices).  The S sorted lists of a row are contiguous ([Q][S][k]),
// so the divide-and-merge (ref. [18]) is one more selection over
// that row of S*k candidates: ties in it fall in position order, which is the
// index order (segments and lists are index-ordered), so the top-k by (value,
// position) is the top-k by (value, index); a gather maps positions to indices.
// ---------------------------------------------------------------------------
struct SplitPlan {
    int S = 1;
    int64_t seg_len = 0;
};

static SplitPlan split_plan(int64_t Q, int64_t N, int k, int sms) {
    SplitPlan p;
    if (Q >= sms) return p;  // a row per SM at least: the direct path streams at full rate
    const int kp = k <= 32 ? 32 : k <= 64 ? 64 : k <= 128 ? 128 : k <= 256 ? 256 : k <= 512 ? 512 : 1024;
    const int64_t min_seg = std::max<int64_t>(32768, 64 * (int64_t)kp);  // each segment >> its k
    // one virtual row per SM at most: each CTA (<= 8 warps, deep ring) then runs in a
    // single wave -- a second, partial wave would double the time
    int64_t S = (int64_t)sms / Q;
    S = std::min<int64_t>(S, N / min_seg);
    if (S < 2) return p;
    p.S = (int)S;
    // equal segments (no alignment rounding: unaligned segment heads are handled in
    // the kernel); the last one holds N - (S-1)*ceil(N/S) >= N/S - S + 1 >> k elements
    p.seg_len = (N + S - 1) / S;
    return p;
}

static size_t split_workspace(const SplitPlan& p, int64_t Q, int k) {
    if (p.S < 2) return 0;
    return 2 * al256((size_t)p.S * (size_t)Q * (size_t)k * 4u) + al256((size_t)Q * (size_t)k * 4u);
}

// out_idx[q][j] = lidx[q][pos[q][j]] (row q of lidx holds S*k indices)
__global__ void split_gather_idx_kernel(const int32_t* __restrict__ lidx, const int32_t* __restrict__ pos,
                                        int64_t Q, int64_t Sk, int k, int32_t* __restrict__ out_idx) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= Q * (int64_t)k) return;
    const int64_t q = t / k;
    out_idx[t] = lidx[q * Sk + pos[t]];
}

size_t ksel_select_workspace(int64_t Q, int64_t N, int k) {
    if (Q < 1 || N < 1 || k < 1 || k > N || k > KSEL_MAX_K) return 0;
    DevInfo di;
    if (current_device_info(&di) != KSEL_OK) return 0;
    return split_workspace(split_plan(Q, N, k, di.sms), Q, k);
}

int ksel_select_ex(const float* dist, int64_t Q, int64_t N, int k, float* out_val, int32_t* out_idx, void* d_work,
                   size_t work_bytes, void* stream) {
    int st = check_select_args(dist, Q, N, k, out_val, out_idx);
    if (st) return st;
    if (!d_work || work_bytes == 0) return ksel_select(dist, Q, N, k, out_val, out_idx, stream);
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    const SplitPlan p = split_plan(Q, N, k, di.sms);
    const size_t need = split_workspace(p, Q, k);
    if (need == 0) return ksel_select(dist, Q, N, k, out_val, out_idx, stream);
    if (work_bytes < need) return KSEL_ERR_INVALID_ARG;
    const size_t in_bytes = (size_t)Q * (size_t)N * 4u, out_bytes = (size_t)Q * (size_t)k * 4u;
    if (overlaps(dist, in_bytes, out_val, out_bytes) || overlaps(dist, in_bytes, out_idx, out_bytes) ||
        overlaps(out_val, out_bytes, out_idx, out_bytes) || overlaps(d_work, need, dist, in_bytes) ||
        overlaps(d_work, need, out_val, out_bytes) || overlaps(d_work, need, out_idx, out_bytes))
        return KSEL_ERR_INVALID_ARG;
    uint8_t* w = static_cast<uint8_t*>(d_work);
    const int64_t Sk = (int64_t)p.S * k;
    const size_t lb = al256((size_t)Q * (size_t)Sk * 4u);
    float* lv = reinterpret_cast<float*>(w);
    int32_t* li = reinterpret_cast<int32_t*>(w + lb);
    int32_t* pos = reinterpret_cast<int32_t*>(w + 2 * lb);
    const cudaStream_t cs = (cudaStream_t)stream;
    const int slot = timing_begin(cs);
    SegMap seg;
    seg.nseg = p.S;
    seg.seg_len = p.seg_len;
    const int64_t V = (int64_t)p.S * Q;  // virtual rows, [Q][S] order
    cudaError_t e = launch_select_pool(dist, V, N, k, lv, li, pool_launch_shape(V, p.seg_len, k, di.sms, 0), cs, seg);
    // second level: top-k of each row's S*k candidates, 8 warps per row (few, short rows)
    if (e == cudaSuccess) e = launch_select_pool(lv, Q, Sk, k, out_val, pos, pool_launch_shape(Q, Sk, k, di.sms, 8), cs);
    if (e == cudaSuccess) {
        const int64_t n = Q * (int64_t)k;
        split_gather_idx_kernel<<<(unsigned)((n + 255) / 256), 256, 0, cs>>>(li, pos, Q, Sk, k, out_idx);
        note_launch();
        e = cudaGetLastError();
    }
    timing_end(slot, cs);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_merge(const float* cand_val, const int32_t* cand_idx, int64_t Q, int S, int kin, int k, float* out_val,
               int32_t* out_idx, void* stream) {
    if (!cand_val || !cand_idx || !out_val || !out_idx) return KSEL_ERR_INVALID_ARG;
    if (Q < 1 || S < 1 || S > 64 || kin < 1 || k < 1 || (int64_t)k > (int64_t)S * kin) return KSEL_ERR_INVALID_ARG;
    if (kin > KSEL_MAX_K || k > KSEL_MAX_K) return KSEL_ERR_UNSUPPORTED;
    const size_t in_b = (size_t)S * (size_t)Q * (size_t)kin * 4u, out_b = (size_t)Q * (size_t)k * 4u;
    if (overlaps(cand_val, in_b, out_val, out_b) || overlaps(cand_val, in_b, out_idx, out_b) ||
        overlaps(cand_idx, in_b, out_val, out_b) || overlaps(cand_idx, in_b, out_idx, out_b) ||
        overlaps(out_val, out_b, out_idx, out_b))
        return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    int st = current_device_info(&di);
    if (st) return st;
    MergeLists L{};
    for (int s = 0; s < S; ++s) {
        L.v[s] = cand_val + (int64_t)s * Q * kin;
        L.i[s] = cand_idx + (int64_t)s * Q * kin;
    }
    cudaError_t e = launch_merge(L, Q, S, kin, k, out_val, out_idx, (cudaStream_t)stream);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

// ---------------------------------------------------------------------------
// host-buffer pipeline (end-to-end entry point)
// ---------------------------------------------------------------------------
static const size_t kHostSlotTarget = 256ull << 20;  // bytes of input per pipeline slot


// bytes of one pipeline slot holding `rows` rows: [dist | out_val | out_idx], 256-B aligned parts
static size_t host_slot_bytes(int64_t rows, int64_t N, int k) {
    return al256((size_t)rows * (size_t)N * 4u) + 2u * al256((size_t)rows * (size_t)k * 4u);
}

static int64_t host_rows_per_slot(int64_t N, int k, size_t work_bytes) {
    int64_t rows = (int64_t)((work_bytes / 2u) / ((size_t)N * 4u + (size_t)k * 8u));
    while (rows > 0 && 2u * host_slot_bytes(rows, N, k) > work_bytes) --rows;
    return rows;
}

size_t ksel_select_host_workspace(int64_t N, int k) {
    if (N < 1 || k < 1) return 0;
    int64_t rows = (int64_t)(kHostSlotTarget / ((size_t)N * 4u));
    if (rows < 1) rows = 1;
    return 2u * host_slot_bytes(rows, N, k);
}

int ksel_select_host(const float* h_dist, int64_t Q, int64_t N, int k, float* h_out_val, int32_t* h_out_idx,
                     void* d_work, size_t work_bytes, void* stream) {
    int st = check_select_args(h_dist, Q, N, k, h_out_val, h_out_idx);
    if (st) return st;
    if (!d_work) return KSEL_ERR_INVALID_ARG;
    const int64_t rps = host_rows_per_slot(N, k, work_bytes);
    if (rps < 1) return KSEL_ERR_INVALID_ARG;
    DevInfo di;
    st = current_device_info(&di);
    if (st) return st;
    const cudaStream_t cs = (cudaStream_t)stream;
    const int64_t rows = rps < Q ? rps : Q;
    const int wpr = pool_launch_shape(rows, N, k, di.sms, 0);

    const size_t dist_b = al256((size_t)rps * (size_t)N * 4u), val_b = al256((size_t)rps * (size_t)k * 4u);
    const size_t slot_b = host_slot_bytes(rps, N, k);
    uint8_t* base = static_cast<uint8_t*>(d_work);
    float* sd[2];
    float* sv[2];
    int32_t* si[2];
    for (int s = 0; s < 2; ++s) {
        uint8_t* p = base + (size_t)s * slot_b;
        sd[s] = reinterpret_cast<float*>(p);
        sv[s] = reinterpret_cast<float*>(p + dist_b);
        si[s] = reinterpret_cast<int32_t*>(p + dist_b + val_b);
    }

    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev_in[2] = {nullptr, nullptr}, ev_comp[2] = {nullptr, nullptr}, ev_out[2] = {nullptr, nullptr};
    cudaEvent_t ev_entry = nullptr;
    cudaError_t e = cudaStreamCreateWithFlags(&h2d, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&d2h, cudaStreamNonBlocking);
    for (int s = 0; s < 2 && e == cudaSuccess; ++s) {
        e = cudaEventCreateWithFlags(&ev_in[s], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev_comp[s], cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev_out[s], cudaEventDisableTiming);
    }
    // Stream order: the copy streams start only after everything already queued on the
    // caller's stream (the workspace may be memory a pending kernel of that stream still
    // uses, e.g. a block just recycled by a caching allocator; a pending D2H copy may still
    // be filling the output host buffers).
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev_entry, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(ev_entry, cs);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(h2d, ev_entry, 0);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(d2h, ev_entry, 0);
    int64_t blk = 0;
    for (int64_t r0 = 0; r0 < Q && e == cudaSuccess; r0 += rows, ++blk) {
        const int s = (int)(blk & 1);
        const int64_t nr = (Q - r0 < rows) ? Q - r0 : rows;
        if (blk >= 2) e = cudaStreamWaitEvent(h2d, ev_comp[s], 0);  // slot input free
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(sd[s], h_dist + r0 * N, (size_t)nr * (size_t)N * 4u, cudaMemcpyHostToDevice, h2d);
        if (e == cudaSuccess) e = cudaEventRecord(ev_in[s], h2d);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, ev_in[s], 0);
        if (e == cudaSuccess && blk >= 2) e = cudaStreamWaitEvent(cs, ev_out[s], 0);  // slot output free
        if (e == cudaSuccess) e = launch_select_pool(sd[s], nr, N, k, sv[s], si[s], wpr, cs);
        if (e == cudaSuccess) e = cudaEventRecord(ev_comp[s], cs);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(d2h, ev_comp[s], 0);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(h_out_val + r0 * k, sv[s], (size_t)nr * (size_t)k * 4u, cudaMemcpyDeviceToHost, d2h);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(h_out_idx + r0 * k, si[s], (size_t)nr * (size_t)k * 4u, cudaMemcpyDeviceToHost, d2h);
        if (e == cudaSuccess) e = cudaEventRecord(ev_out[s], d2h);
    }
    if (e == cudaSuccess) {
        e = cudaStreamSynchronize(d2h);
    } else {
        // error path: no copy may still touch the caller's host buffers after return
        if (h2d) cudaStreamSynchronize(h2d);
        cudaStreamSynchronize(cs);
        if (d2h) cudaStreamSynchronize(d2h);
    }
    if (ev_entry) cudaEventDestroy(ev_entry);
    for (int s = 0; s < 2; ++s) {
        if (ev_in[s]) cudaEventDestroy(ev_in[s]);
        if (ev_comp[s]) cudaEventDestroy(ev_comp[s]);
        if (ev_out[s]) cudaEventDestroy(ev_out[s]);
    }
    if (h2d) cudaStreamDestroy(h2d);
    if (d2h) cudaStreamDestroy(d2h);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

// knn_search: declared for the ABI; the fused tcgen05 path lives in knn_fused.cu.
}  // extern "C"
