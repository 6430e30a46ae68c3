"""B200-native batched k-selection (Tang et al., IPDPS 2015) -- Python binding.

Thin ctypes marshalling over the C ABI of ``libksel.so`` (``include/ksel.h``):
every step of the hot path runs in the library's sm_100a kernels.  PyTorch is
used only for device memory and the current CUDA stream.  There is no CPU or
library fallback: if ``libksel.so`` is missing this module raises on import.

Entry points (same names as the C ABI):

* :func:`ksel_select`      -- k smallest (value, index) pairs of every row.
* :func:`ksel_select_host` -- the same on host buffers (end-to-end path).
* :func:`ksel_merge`       -- top-k of the union of S sorted candidate lists.
* :func:`knn_search`       -- fused distance + selection brute-force k-NN.
* :func:`knn_graph`        -- k-NN graph of one point set (self excluded).
* :func:`ksel_select_paper` -- ABLATION: the paper's per-thread queue / buffer / HP
  designs (query-contiguous input), bit-identical results.
* :func:`ksel_merge_lists` -- ksel_merge over pointer tables (peer lists, ready flags);
  with :func:`ipc_alloc` / :func:`ipc_open` / :func:`flag_signal` / :func:`flag_wait`
  the collective-free row-sharded k-NN exchange (dist.KnnP2P).
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libksel.so")
# tools/ timing experiments only: load the -DKSEL_EXPERIMENTS build (libksel_exp.so), or
# an A/B build of another revision (KSEL_AB_LIB=<file name next to this one>)
if os.environ.get("KSEL_EXPERIMENTS_LIB") == "1":
    LIB_PATH = os.path.join(_HERE, "libksel_exp.so")
elif os.environ.get("KSEL_AB_LIB"):
    LIB_PATH = os.path.join(_HERE, os.path.basename(os.environ["KSEL_AB_LIB"]))

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libksel.so is not built (expected at %s); run `python __graft_entry__.py` "
        "or paper_conf_ipps_tang0emg15_b200/build.py" % LIB_PATH)

_lib = ctypes.CDLL(LIB_PATH)
_p, _i64, _i32, _sz = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_size_t
_lib.ksel_select.argtypes = [_p, _i64, _i64, _i32, _p, _p, _p]
_lib.ksel_select_config.argtypes = [_p, _i64, _i64, _i32, _p, _p, _i32, _i32, _p]
_lib.ksel_select_workspace.argtypes = [_i64, _i64, _i32]
_lib.ksel_select_workspace.restype = _sz
_lib.ksel_select_ex.argtypes = [_p, _i64, _i64, _i32, _p, _p, _p, _sz, _p]
_lib.ksel_select_ex.restype = ctypes.c_int
_lib.ksel_select_host_workspace.argtypes = [_i64, _i32]
_lib.ksel_select_host_workspace.restype = _sz
_lib.ksel_select_host.argtypes = [_p, _i64, _i64, _i32, _p, _p, _p, _sz, _p]
_lib.ksel_merge.argtypes = [_p, _p, _i64, _i32, _i32, _i32, _p, _p, _p]
_lib.knn_search_workspace.argtypes = [_i64, _i64, _i32, _i32]
_lib.knn_search_workspace.restype = _sz
_lib.knn_search.argtypes = [_p, _p, _i64, _i64, _i32, _i32, _p, _p, _i64, _p, _sz, _p]
_lib.knn_graph_workspace.argtypes = [_i64, _i32, _i32]
_lib.knn_graph_workspace.restype = _sz
_lib.knn_graph.argtypes = [_p, _i64, _i32, _i32, _p, _p, _p, _sz, _p]
_lib.knn_graph.restype = ctypes.c_int
_lib.knn_distances_workspace.argtypes = [_i64, _i64, _i32]
_lib.knn_distances_workspace.restype = _sz
_lib.knn_distances.argtypes = [_p, _p, _i64, _i64, _i32, _p, _p, _p, _sz, _p]
_lib.knn_distances.restype = ctypes.c_int
_lib.ksel_timing_enable.argtypes = [_i32]
_lib.ksel_timing_enable.restype = ctypes.c_int
_lib.ksel_timing_collect.argtypes = [ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64)]
_lib.ksel_timing_collect.restype = ctypes.c_int
_lib.ksel_strerror.argtypes = [_i32]
_lib.ksel_strerror.restype = ctypes.c_char_p
_lib.ksel_launch_count.restype = _i64
_lib.ksel_select_paper_workspace.argtypes = [_i64, _i64, _i32, _i32, _i32, _i32, _i32, _i32]
_lib.ksel_select_paper_workspace.restype = _sz
_lib.ksel_select_paper.argtypes = [_p, _i64, _i64, _i32, _i32, _i32, _i32, _i32, _i32, _p, _p, _p, _sz, _p]
_lib.ksel_select_paper.restype = ctypes.c_int
_lib.ksel_ipc_handle_size.restype = _sz
_lib.ksel_ipc_alloc.argtypes = [_sz, ctypes.POINTER(ctypes.c_void_p), _p]
_lib.ksel_ipc_open.argtypes = [_p, ctypes.POINTER(ctypes.c_void_p)]
_lib.ksel_ipc_close.argtypes = [_p]
_lib.ksel_ipc_free.argtypes = [_p]
_lib.ksel_flag_signal.argtypes = [_p, ctypes.c_uint32, _p]
_lib.ksel_flag_wait.argtypes = [_p, _i32, ctypes.c_uint32, _p]
_lib.ksel_merge_lists.argtypes = [_p, _p, _i32, _i64, _i32, _i32, _p, _p, _p, ctypes.c_uint32, _p]
_lib.ksel_set_flag_timeout.argtypes = [ctypes.c_double]
for _f in (_lib.ksel_ipc_alloc, _lib.ksel_ipc_open, _lib.ksel_ipc_close, _lib.ksel_ipc_free, _lib.ksel_flag_signal,
           _lib.ksel_flag_wait, _lib.ksel_merge_lists, _lib.ksel_set_flag_timeout, _lib.ksel_device_status,
           _lib.ksel_device_status_clear):
    _f.restype = ctypes.c_int
for _f in (_lib.ksel_select, _lib.ksel_select_config, _lib.ksel_select_host, _lib.ksel_merge, _lib.knn_search, _lib.ksel_version):
    _f.restype = ctypes.c_int

KSEL_MAX_K = 1024
ALGO_AUTO, ALGO_QUEUE, ALGO_POOL, ALGO_RADIX, ALGO_HIST = 0, 1, 2, 3, 4
PQ_INSERT, PQ_HEAP, PQ_MERGE, PQ_MERGE_ALIGNED = 0, 1, 2, 3
PB_NONE, PB_BUFFER, PB_FULL, PB_FULL_SORTED = 0, 1, 2, 3
EXPORTS = ("ksel_select", "ksel_select_workspace", "ksel_select_ex", "ksel_select_config", "ksel_select_host_workspace", "ksel_select_host", "ksel_merge",
           "knn_search_workspace", "knn_search", "knn_graph_workspace", "knn_graph", "knn_distances_workspace", "knn_distances", "ksel_timing_enable", "ksel_timing_collect", "ksel_strerror",
           "ksel_version", "ksel_launch_count", "ksel_select_paper_workspace", "ksel_select_paper", "ksel_ipc_handle_size", "ksel_ipc_alloc", "ksel_ipc_open",
           "ksel_ipc_close", "ksel_ipc_free", "ksel_flag_signal", "ksel_flag_wait", "ksel_merge_lists",
           "ksel_set_flag_timeout", "ksel_device_status", "ksel_device_status_clear")


class KselError(RuntimeError):
    def __init__(self, fn: str, status: int):
        self.status = status
        super().__init__("%s failed: %s (status %d)" % (fn, strerror(status), status))


def strerror(status: int) -> str:
    return _lib.ksel_strerror(status).decode()


def version() -> int:
    return _lib.ksel_version()


def launch_count() -> int:
    """Kernels enqueued by libksel since load (all entry points)."""
    return _lib.ksel_launch_count()


def timing_enable(on: bool = True) -> None:
    """Record CUDA events around the dominant kernel of every call (bench.py)."""
    _lib.ksel_timing_enable(1 if on else 0)


def timing_collect():
    """(total milliseconds, launches) of the dominant kernels timed since the last collect."""
    ms, n = ctypes.c_double(0.0), ctypes.c_int64(0)
    _check("ksel_timing_collect", _lib.ksel_timing_collect(ctypes.byref(ms), ctypes.byref(n)))
    return ms.value, n.value


def _check(fn, status):
    if status != 0:
        raise KselError(fn, status)


def _dev_f32(t: torch.Tensor, name: str, ndim: int):
    if not isinstance(t, torch.Tensor) or t.device.type != "cuda":
        raise TypeError("%s must be a CUDA tensor" % name)
    if t.dtype != torch.float32 or t.dim() != ndim or not t.is_contiguous():
        raise TypeError("%s must be a contiguous %d-D float32 tensor" % (name, ndim))


def _stream(device) -> int:
    return torch.cuda.current_stream(device).cuda_stream


def _out(t, name: str, shape, dtype, device):
    """A caller-supplied output: exact shape, dtype, contiguous, on `device` (the kernels
    write every element through the raw pointer, so a mismatch would corrupt memory)."""
    if not isinstance(t, torch.Tensor):
        raise TypeError("%s must be a tensor" % name)
    if tuple(t.shape) != tuple(shape) or t.dtype != dtype or not t.is_contiguous() or t.device != device:
        raise TypeError("%s must be a contiguous %s tensor of shape %s on %s (got %s %s on %s%s)"
                        % (name, dtype, tuple(shape), device, t.dtype, tuple(t.shape), t.device,
                           "" if t.is_contiguous() else ", non-contiguous"))


def _workspace(ws, need: int, device, name: str = "workspace"):
    if not isinstance(ws, torch.Tensor) or ws.device != device or not ws.is_contiguous():
        raise TypeError("%s must be a contiguous tensor on %s" % (name, device))
    if ws.numel() * ws.element_size() < need:
        raise ValueError("%s holds %d bytes, %d needed" % (name, ws.numel() * ws.element_size(), need))


def _same_device(a: torch.Tensor, b: torch.Tensor, an: str, bn: str):
    if a.device != b.device:
        raise ValueError("%s and %s must be on the same device (%s vs %s)" % (an, bn, a.device, b.device))


def ksel_select_workspace(Q: int, N: int, k: int) -> int:
    return int(_lib.ksel_select_workspace(Q, N, k))


def ksel_select(dist: torch.Tensor, k: int, out_val: torch.Tensor | None = None,
                out_idx: torch.Tensor | None = None, algo: int = ALGO_AUTO, warps_per_row: int = 0,
                workspace: torch.Tensor | None = None, split_rows: bool = True):
    """k smallest (value, index) pairs per row of ``dist`` [Q, N], ascending.

    Returns (values float32 [Q, k] with the input bits, indices int32 [Q, k]).
    Enqueued on the current stream; asynchronous.  ``algo``/``warps_per_row``
    pin the kernel variant (ksel_select_config); defaults pick automatically.
    With the defaults, few long rows go through ksel_select_ex (split rows) with
    ``workspace`` (allocated here when None and needed); ``split_rows=False``
    forces the one-CTA-per-row path."""
    _dev_f32(dist, "dist", 2)
    Q, N = dist.shape
    if out_val is None:
        out_val = torch.empty((Q, k), dtype=torch.float32, device=dist.device)
    _out(out_val, "out_val", (Q, k), torch.float32, dist.device)
    if out_idx is None:
        out_idx = torch.empty((Q, k), dtype=torch.int32, device=dist.device)
    _out(out_idx, "out_idx", (Q, k), torch.int32, dist.device)
    with torch.cuda.device(dist.device):
        need = ksel_select_workspace(Q, N, k) if (algo == ALGO_AUTO and warps_per_row == 0 and split_rows) else 0
        if need > 0:
            if workspace is None:
                workspace = torch.empty(need, dtype=torch.uint8, device=dist.device)
            _workspace(workspace, need, dist.device)
            st = _lib.ksel_select_ex(dist.data_ptr(), Q, N, k, out_val.data_ptr(), out_idx.data_ptr(),
                                     workspace.data_ptr(), workspace.numel() * workspace.element_size(),
                                     _stream(dist.device))
        elif algo == ALGO_AUTO and warps_per_row == 0:
            st = _lib.ksel_select(dist.data_ptr(), Q, N, k, out_val.data_ptr(), out_idx.data_ptr(),
                                  _stream(dist.device))
        else:
            st = _lib.ksel_select_config(dist.data_ptr(), Q, N, k, out_val.data_ptr(), out_idx.data_ptr(),
                                         algo, warps_per_row, _stream(dist.device))
        _check("ksel_select", st)
    return out_val, out_idx


def ksel_select_host_workspace(N: int, k: int) -> int:
    return int(_lib.ksel_select_host_workspace(N, k))


def ksel_select_host(dist: torch.Tensor, k: int, out_val: torch.Tensor | None = None,
                     out_idx: torch.Tensor | None = None, workspace: torch.Tensor | None = None,
                     device=None):
    """End-to-end selection on HOST tensors (pin them for overlapped copies).

    ``dist`` is a contiguous float32 CPU tensor [Q, N]; results are CPU tensors.
    The call returns when the results are in host memory."""
    if dist.device.type != "cpu" or dist.dtype != torch.float32 or not dist.is_contiguous():
        raise TypeError("dist must be a contiguous float32 CPU tensor")
    Q, N = dist.shape
    dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
    if out_val is None:
        out_val = torch.empty((Q, k), dtype=torch.float32, pin_memory=dist.is_pinned())
    _out(out_val, "out_val", (Q, k), torch.float32, torch.device("cpu"))
    if out_idx is None:
        out_idx = torch.empty((Q, k), dtype=torch.int32, pin_memory=dist.is_pinned())
    _out(out_idx, "out_idx", (Q, k), torch.int32, torch.device("cpu"))
    if workspace is None:
        workspace = torch.empty(ksel_select_host_workspace(N, k), dtype=torch.uint8, device=dev)
    if workspace.device.type != "cuda" or not workspace.is_contiguous():
        raise TypeError("workspace must be a contiguous CUDA tensor")
    dev = workspace.device
    with torch.cuda.device(dev):
        _check("ksel_select_host", _lib.ksel_select_host(
            dist.data_ptr(), Q, N, k, out_val.data_ptr(), out_idx.data_ptr(), workspace.data_ptr(),
            workspace.numel() * workspace.element_size(), _stream(dev)))
    return out_val, out_idx


def ksel_merge(cand_val: torch.Tensor, cand_idx: torch.Tensor, k: int,
               out_val: torch.Tensor | None = None, out_idx: torch.Tensor | None = None):
    """Top-k of the union of S sorted lists per query; inputs are [S, Q, kin]."""
    _dev_f32(cand_val, "cand_val", 3)
    if cand_idx.dtype != torch.int32 or cand_idx.shape != cand_val.shape or not cand_idx.is_contiguous():
        raise TypeError("cand_idx must be a contiguous int32 tensor shaped like cand_val")
    _same_device(cand_val, cand_idx, "cand_val", "cand_idx")
    S, Q, kin = cand_val.shape
    if out_val is None:
        out_val = torch.empty((Q, k), dtype=torch.float32, device=cand_val.device)
    _out(out_val, "out_val", (Q, k), torch.float32, cand_val.device)
    if out_idx is None:
        out_idx = torch.empty((Q, k), dtype=torch.int32, device=cand_val.device)
    _out(out_idx, "out_idx", (Q, k), torch.int32, cand_val.device)
    with torch.cuda.device(cand_val.device):
        _check("ksel_merge", _lib.ksel_merge(cand_val.data_ptr(), cand_idx.data_ptr(), Q, S, kin, k,
                                             out_val.data_ptr(), out_idx.data_ptr(),
                                             _stream(cand_val.device)))
    return out_val, out_idx


def knn_search_workspace(N: int, Q: int, D: int, k: int) -> int:
    return int(_lib.knn_search_workspace(N, Q, D, k))


def knn_search(ref: torch.Tensor, query: torch.Tensor, k: int, idx_offset: int = 0,
               out_dist: torch.Tensor | None = None, out_idx: torch.Tensor | None = None,
               workspace: torch.Tensor | None = None):
    """k nearest references (squared L2) of every query; ref [N, D], query [Q, D]."""
    _dev_f32(ref, "ref", 2)
    _dev_f32(query, "query", 2)
    _same_device(ref, query, "ref", "query")
    N, D = ref.shape
    Q = query.shape[0]
    if query.shape[1] != D:
        raise ValueError("ref and query must share D")
    if out_dist is None:
        out_dist = torch.empty((Q, k), dtype=torch.float32, device=ref.device)
    _out(out_dist, "out_dist", (Q, k), torch.float32, ref.device)
    if out_idx is None:
        out_idx = torch.empty((Q, k), dtype=torch.int32, device=ref.device)
    _out(out_idx, "out_idx", (Q, k), torch.int32, ref.device)
    need = knn_search_workspace(N, Q, D, k)
    if workspace is None and need > 0:
        workspace = torch.empty(need, dtype=torch.uint8, device=ref.device)
    if workspace is not None:
        _workspace(workspace, need, ref.device)
    wptr = workspace.data_ptr() if workspace is not None else 0
    wlen = workspace.numel() * workspace.element_size() if workspace is not None else 0
    with torch.cuda.device(ref.device):
        _check("knn_search", _lib.knn_search(ref.data_ptr(), query.data_ptr(), N, Q, D, k,
                                             out_dist.data_ptr(), out_idx.data_ptr(), idx_offset,
                                             wptr, wlen, _stream(ref.device)))
    return out_dist, out_idx


def knn_graph_workspace(N: int, D: int, k: int) -> int:
    return int(_lib.knn_graph_workspace(N, D, k))


def knn_graph(points: torch.Tensor, k: int, out_dist: torch.Tensor | None = None,
              out_idx: torch.Tensor | None = None, workspace: torch.Tensor | None = None):
    """k nearest OTHER points of every point (k-NN graph); points [N, D]."""
    _dev_f32(points, "points", 2)
    N, D = points.shape
    if out_dist is None:
        out_dist = torch.empty((N, k), dtype=torch.float32, device=points.device)
    _out(out_dist, "out_dist", (N, k), torch.float32, points.device)
    if out_idx is None:
        out_idx = torch.empty((N, k), dtype=torch.int32, device=points.device)
    _out(out_idx, "out_idx", (N, k), torch.int32, points.device)
    need = knn_graph_workspace(N, D, k)
    if workspace is None and need > 0:
        workspace = torch.empty(need, dtype=torch.uint8, device=points.device)
    if workspace is not None:
        _workspace(workspace, need, points.device)
    wptr = workspace.data_ptr() if workspace is not None else 0
    wlen = workspace.numel() * workspace.element_size() if workspace is not None else 0
    with torch.cuda.device(points.device):
        _check("knn_graph", _lib.knn_graph(points.data_ptr(), N, D, k, out_dist.data_ptr(), out_idx.data_ptr(),
                                           wptr, wlen, _stream(points.device)))
    return out_dist, out_idx


def knn_distances(ref: torch.Tensor, query: torch.Tensor, out: torch.Tensor | None = None, with_eps: bool = False):
    """DIAGNOSTIC: the tensor-core filter distances d~ [Q, N] (materialised); with_eps
    also returns the per-query bound eps [Q] with |d~ - d| <= eps."""
    _dev_f32(ref, "ref", 2)
    _dev_f32(query, "query", 2)
    N, D = ref.shape
    Q = query.shape[0]
    _same_device(ref, query, "ref", "query")
    if out is None:
        out = torch.empty((Q, N), dtype=torch.float32, device=ref.device)
    _out(out, "out", (Q, N), torch.float32, ref.device)
    eps = torch.empty(Q, dtype=torch.float32, device=ref.device) if with_eps else None
    ws = torch.empty(max(1, int(_lib.knn_distances_workspace(N, Q, D))), dtype=torch.uint8, device=ref.device)
    with torch.cuda.device(ref.device):
        _check("knn_distances", _lib.knn_distances(ref.data_ptr(), query.data_ptr(), N, Q, D, out.data_ptr(),
                                                   eps.data_ptr() if with_eps else None, ws.data_ptr(),
                                                   ws.numel(), _stream(ref.device)))
    return (out, eps) if with_eps else out


# ---- collective-free exchange (ksel_ipc_*, ksel_flag_*, ksel_merge_lists) ----

class _CudaMem:
    """__cuda_array_interface__ over a raw device pointer (no ownership)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 2, "strides": None}


def device_bytes(ptr: int, nbytes: int) -> torch.Tensor:
    """A uint8 CUDA tensor viewing [ptr, ptr + nbytes) of the current device (no copy)."""
    return torch.as_tensor(_CudaMem(ptr, nbytes), device="cuda")


def ipc_alloc(nbytes: int):
    """(device pointer, handle bytes) of a fresh zero-filled exportable allocation."""
    h = ctypes.create_string_buffer(int(_lib.ksel_ipc_handle_size()))
    p = ctypes.c_void_p()
    _check("ksel_ipc_alloc", _lib.ksel_ipc_alloc(nbytes, ctypes.byref(p), h))
    return int(p.value), bytes(h.raw)


def ipc_open(handle: bytes) -> int:
    p = ctypes.c_void_p()
    _check("ksel_ipc_open", _lib.ksel_ipc_open(handle, ctypes.byref(p)))
    return int(p.value)


def ipc_close(ptr: int) -> None:
    _check("ksel_ipc_close", _lib.ksel_ipc_close(ptr))


def ipc_free(ptr: int) -> None:
    _check("ksel_ipc_free", _lib.ksel_ipc_free(ptr))


def _ptr_array(ptrs):
    return (ctypes.c_void_p * len(ptrs))(*[int(x) for x in ptrs])


def flag_signal(flag_ptr: int, value: int) -> None:
    """Stream-ordered release store of `value` to a u32 flag (local or peer memory)."""
    _check("ksel_flag_signal", _lib.ksel_flag_signal(flag_ptr, value & 0xFFFFFFFF,
                                                     torch.cuda.current_stream().cuda_stream))


def flag_wait(flag_ptrs, value: int) -> None:
    """Later work on the current stream waits until every flag reached `value`."""
    arr = _ptr_array(flag_ptrs)
    _check("ksel_flag_wait", _lib.ksel_flag_wait(arr, len(flag_ptrs), value & 0xFFFFFFFF,
                                                 torch.cuda.current_stream().cuda_stream))


def set_flag_timeout(seconds: float) -> None:
    """Timeout of device-side flag waits enqueued from now on (default 600 s)."""
    _check("ksel_set_flag_timeout", _lib.ksel_set_flag_timeout(float(seconds)))


def device_status() -> int:
    """0, or 5 (KSEL_ERR_TIMEOUT) if a device-side flag wait gave up since the last clear.
    Synchronise the stream(s) first."""
    return int(_lib.ksel_device_status())


def device_status_clear() -> None:
    _lib.ksel_device_status_clear()


def ksel_merge_lists(val_ptrs, idx_ptrs, Q: int, kin: int, k: int, out_val: torch.Tensor, out_idx: torch.Tensor,
                     ready_ptrs=None, epoch: int = 0):
    """ksel_merge over pointer tables: list s of query q at val_ptrs[s] + 4*q*kin (device pointers)."""
    S = len(val_ptrs)
    if len(idx_ptrs) != S or (ready_ptrs is not None and len(ready_ptrs) != S):
        raise ValueError("pointer tables differ in length")
    if out_val.shape != (Q, k) or out_idx.shape != (Q, k) or out_val.dtype != torch.float32 \
            or out_idx.dtype != torch.int32 or not out_val.is_contiguous() or not out_idx.is_contiguous():
        raise TypeError("out_val/out_idx must be contiguous [Q, k] float32/int32 tensors")
    rd = _ptr_array(ready_ptrs) if ready_ptrs is not None else None
    _check("ksel_merge_lists", _lib.ksel_merge_lists(_ptr_array(val_ptrs), _ptr_array(idx_ptrs), S, Q, kin, k,
                                                     out_val.data_ptr(), out_idx.data_ptr(), rd,
                                                     epoch & 0xFFFFFFFF, torch.cuda.current_stream().cuda_stream))
    return out_val, out_idx


def ksel_select_paper(dist_t: torch.Tensor, k: int, queue: int = PQ_MERGE_ALIGNED, buffer: int = PB_FULL_SORTED,
                      hp_G: int = 4, m: int = 8, bsize: int = 16, workspace: torch.Tensor | None = None):
    """ABLATION: the paper's thread-per-query designs.  dist_t is [N, Q]
    (query-contiguous: column q is query q's row); returns ([Q, k] values, [Q, k] indices)."""
    _dev_f32(dist_t, "dist_t", 2)
    N, Q = dist_t.shape
    need = int(_lib.ksel_select_paper_workspace(Q, N, k, queue, buffer, hp_G, m, bsize))
    if need == 0:
        raise KselError("ksel_select_paper_workspace", 1)
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device=dist_t.device)
    ov = torch.empty((Q, k), dtype=torch.float32, device=dist_t.device)
    oi = torch.empty((Q, k), dtype=torch.int32, device=dist_t.device)
    with torch.cuda.device(dist_t.device):
        _check("ksel_select_paper", _lib.ksel_select_paper(dist_t.data_ptr(), Q, N, k, queue, buffer, hp_G, m, bsize,
                                                           ov.data_ptr(), oi.data_ptr(), workspace.data_ptr(),
                                                           workspace.numel(), _stream(dist_t.device)))
    return ov, oi
