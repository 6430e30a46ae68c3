// p2p.cu -- the row-sharded k-NN's exchange without a collective.
//
// After each rank's knn_search (its reference shard, global indices), rank r
// needs, for its slice of queries, the S = world per-shard top-k lists -- the
// divide-and-merge of PAPER.md L243.  Instead of an NCCL all-gather of every
// rank's Q*k candidates followed by ksel_merge, the merge kernel reads the
// peers' candidate lists in place, over NVLink / NVSwitch peer memory (CUDA IPC
// mappings): each rank pulls only the (Q/g)*k*g pairs it merges, and the
// exchange is stream-ordered device-side signalling, no host round trip:
//
//   producer:  knn_search -> buffer[e % 2];  ksel_flag_signal(ready[e % 2] = e + 1)
//   consumer:  ksel_merge_lists(peer lists, ready flags, epoch e + 1)   (each warp
//              waits for a list's flag, acquire at system scope, then reads it
//              with volatile loads);  ksel_flag_signal(peer's consumed[rank] = e + 1)
//   reuse:     before writing buffer[e % 2] again (step e + 2) the producer's stream
//              waits (ksel_flag_wait) until every consumer published consumed >= e + 1.
//
// The library only provides the mechanism (IPC allocation / mapping, release /
// acquire flags, the pointer-table merge); the orchestration lives in
// paper_conf_ipps_tang0emg15_b200/dist.py (KnnP2P).
#include <cstdint>
#include <atomic>
#include <cstring>
#include <mutex>

#include <cuda_runtime.h>

#include "ksel.h"
#include "ksel_common.cuh"
#include "ksel_internal.h"

namespace ksel {

__global__ void flag_signal_kernel(uint32_t* flag, uint32_t value) {
    // every write of earlier kernels in the stream is complete (stream order);
    // make them visible system-wide before the flag (release at system scope)
    __threadfence_system();
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flag), "r"(value) : "memory");
}

struct FlagSet {
    const uint32_t* f[kMaxLists];
};

__global__ void flag_wait_kernel(const __grid_constant__ FlagSet fs, int n, uint32_t value, uint32_t* err,
                                 uint64_t timeout_ns) {
    const int j = (int)threadIdx.x;
    if (j < n) {
        uint32_t v;
        const uint64_t t0 = globaltimer_ns();
        while (true) {
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(fs.f[j]) : "memory");
            if ((int32_t)(v - value) >= 0) break;
            __nanosleep(500);
            if (globaltimer_ns() - t0 > timeout_ns) {  // a peer that never signals: give up, report
                note_timeout(err);
                break;
            }
        }
    }
    __syncthreads();
    __threadfence_system();
}

static std::mutex g_err_mu;
static uint32_t* g_err_host = nullptr;  // mapped pinned host word (written by the device)
static uint32_t* g_err_dev = nullptr;
static std::atomic<uint64_t> g_timeout_ns{600ull * 1000000000ull};

uint32_t* device_error_word() {
    std::lock_guard<std::mutex> lock(g_err_mu);
    if (!g_err_dev) {
        void* h = nullptr;
        if (cudaHostAlloc(&h, 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) return nullptr;
        void* d = nullptr;
        if (cudaHostGetDevicePointer(&d, h, 0) != cudaSuccess) {
            cudaFreeHost(h);
            return nullptr;
        }
        static_cast<volatile uint32_t*>(h)[0] = 0u;
        g_err_host = static_cast<uint32_t*>(h);
        g_err_dev = static_cast<uint32_t*>(d);
    }
    return g_err_dev;
}

uint64_t flag_timeout_ns() { return g_timeout_ns.load(std::memory_order_relaxed); }

}  // namespace ksel

using namespace ksel;

extern "C" {

int ksel_set_flag_timeout(double seconds) {
    if (!(seconds > 0.0) || seconds > 1e9) return KSEL_ERR_INVALID_ARG;
    g_timeout_ns.store((uint64_t)(seconds * 1e9), std::memory_order_relaxed);
    return KSEL_OK;
}

int ksel_device_status(void) {
    std::lock_guard<std::mutex> lock(g_err_mu);
    if (!g_err_host) return KSEL_OK;
    return (static_cast<volatile uint32_t*>(g_err_host)[0] != 0u) ? KSEL_ERR_TIMEOUT : KSEL_OK;
}

int ksel_device_status_clear(void) {
    std::lock_guard<std::mutex> lock(g_err_mu);
    if (g_err_host) static_cast<volatile uint32_t*>(g_err_host)[0] = 0u;
    return KSEL_OK;
}

size_t ksel_ipc_handle_size(void) { return sizeof(cudaIpcMemHandle_t); }

int ksel_ipc_alloc(size_t bytes, void** d_ptr, void* handle_out) {
    if (!d_ptr || !handle_out || bytes == 0) return KSEL_ERR_INVALID_ARG;
    *d_ptr = nullptr;
    void* p = nullptr;
    if (cudaMalloc(&p, bytes) != cudaSuccess) return KSEL_ERR_CUDA;
    if (cudaMemset(p, 0, bytes) != cudaSuccess) { cudaFree(p); return KSEL_ERR_CUDA; }
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, p) != cudaSuccess) { cudaFree(p); return KSEL_ERR_CUDA; }
    std::memcpy(handle_out, &h, sizeof(h));
    *d_ptr = p;
    return KSEL_OK;
}

int ksel_ipc_open(const void* handle, void** d_ptr) {
    if (!handle || !d_ptr) return KSEL_ERR_INVALID_ARG;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, sizeof(h));
    *d_ptr = nullptr;
    return cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess) == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_ipc_close(void* d_ptr) {
    if (!d_ptr) return KSEL_ERR_INVALID_ARG;
    return cudaIpcCloseMemHandle(d_ptr) == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_ipc_free(void* d_ptr) {
    if (!d_ptr) return KSEL_ERR_INVALID_ARG;
    return cudaFree(d_ptr) == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_flag_signal(uint32_t* d_flag, uint32_t value, void* stream) {
    if (!d_flag || (reinterpret_cast<uintptr_t>(d_flag) & 3u)) return KSEL_ERR_INVALID_ARG;
    flag_signal_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(d_flag, value);
    note_launch();
    return cudaGetLastError() == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_flag_wait(const uint32_t* const* d_flags, int n, uint32_t value, void* stream) {
    if (!d_flags || n < 1 || n > kMaxLists) return KSEL_ERR_INVALID_ARG;
    FlagSet fs{};
    for (int j = 0; j < n; ++j) {
        if (!d_flags[j] || (reinterpret_cast<uintptr_t>(d_flags[j]) & 3u)) return KSEL_ERR_INVALID_ARG;
        fs.f[j] = d_flags[j];
    }
    flag_wait_kernel<<<1, 64, 0, (cudaStream_t)stream>>>(fs, n, value, device_error_word(), flag_timeout_ns());
    note_launch();
    return cudaGetLastError() == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

int ksel_merge_lists(const float* const* vals, const int32_t* const* idxs, int S, int64_t Q, int kin, int k,
                     float* out_val, int32_t* out_idx, const uint32_t* const* ready, uint32_t epoch, void* stream) {
    if (!vals || !idxs || !out_val || !out_idx) return KSEL_ERR_INVALID_ARG;
    if (Q < 1 || S < 1 || S > kMaxLists || kin < 1 || k < 1 || (int64_t)k > (int64_t)S * kin)
        return KSEL_ERR_INVALID_ARG;
    if (kin > KSEL_MAX_K || k > KSEL_MAX_K) return KSEL_ERR_UNSUPPORTED;
    MergeLists L{};
    for (int s = 0; s < S; ++s) {
        if (!vals[s] || !idxs[s]) return KSEL_ERR_INVALID_ARG;
        if ((reinterpret_cast<uintptr_t>(vals[s]) & 3u) || (reinterpret_cast<uintptr_t>(idxs[s]) & 3u))
            return KSEL_ERR_INVALID_ARG;
        L.v[s] = vals[s];
        L.i[s] = idxs[s];
        L.ready[s] = ready ? ready[s] : nullptr;
        if (ready && !ready[s]) return KSEL_ERR_INVALID_ARG;
    }
    L.epoch = epoch;
    L.vol = ready ? 1 : 0;
    L.err = ready ? device_error_word() : nullptr;
    L.timeout_ns = flag_timeout_ns();
    DevInfo di;
    int st = current_device_info(&di);
    if (st) return st;
    cudaError_t e = launch_merge(L, Q, S, kin, k, out_val, out_idx, (cudaStream_t)stream);
    return e == cudaSuccess ? KSEL_OK : KSEL_ERR_CUDA;
}

}  // extern "C"
