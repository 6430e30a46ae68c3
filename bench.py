#!/usr/bin/env python
"""bench.py -- batched k-selection throughput on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...

Workload (BASELINE.json configs[2], the 1/2/4/8-GPU config): ksel_select over
Q = 16384 rows in total of N = 2^20 uniform fp32 distances, k = 256,
query-sharded (rank r owns global rows [r*Q/g, (r+1)*Q/g); no communication;
strong scaling by default -- the total work is fixed, as configs[2] states;
--scaling weak keeps 16384 rows per rank).  A step is one ksel_select call
over the rank's rows, inputs resident in HBM (64 GiB at g = 1, far larger than
the 126 MB L2, so no flush is needed between steps).  Metric: selected rows/s
(whole job) and achieved HBM GB/s vs the measured peak.

At N = 1 the same JSON line also carries a `sweep`: the north star's k sweep
(BASELINE configs[1]: Q = 1024, N = 65536, k in {1, 8, 32, 128, 256, 1024} on
uniform / Gaussian / sorted ascending / sorted descending / tied rows), the
fused kNN of configs[3] (C4) and the per-rank shape of configs[4] (C5: N = 10^6
references, Q = 10^4, k = 1024), each as device time, throughput and roofline
fraction.

Rank 0 prints ONE JSON line.  --impl reference times the CPU oracle (oracle/)
on this host's cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "selected rows/sec and achieved HBM GB/s vs peak for Q×N,k at 1/2/4/8 B200"
CONFIGS = {
    # name: (Q per rank, N, k, distribution)
    "c3": (16384, 1 << 20, 256, "U"),
    "c2": (1024, 65536, 256, "U"),
    "c1": (16, 4096, 32, "U"),
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", choices=["c1", "c2", "c3", "c4", "c5"], default="c3")
    ap.add_argument("--k", type=int, default=None)
    ap.add_argument("--dist", default=None)
    ap.add_argument("--scaling", choices=["weak", "strong"], default="strong")
    ap.add_argument("--no-sweep", action="store_true", help="skip the k x distribution / kNN sweep (N = 1)")
    ap.add_argument("--knn-sharded", choices=["auto", "on", "off"], default="auto",
                    help="also time the row-sharded kNN (configs[4]) over the process group: "
                         "auto = only when N > 1")
    ap.add_argument("--e2e-rows", type=int, default=0,
                    help="rows per end-to-end step per rank (host buffers); 0 = 2048 on one GPU, "
                         "512 per rank on several (pinned host memory: 4 MB per row)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--cpu-sample-rows", type=int, default=0, help="0 = auto (~10-30 s of CPU work)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    return ap.parse_args()


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_traffic(workload: str):
    """dram bytes per launch of the dominant kernel from the committed ncu capture."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f).get(workload)
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks/throttle sampling while the timed region runs."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), "--query-gpu=" + self.FIELDS, "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for name, val in zip(names, parts[5:9]):
                if val.lower() == "active":
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def cpu_count():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def cpu_info():
    """Host CPU model and socket count (lscpu), for the cpu_baseline record."""
    model, sockets = None, None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            key, _, val = ln.partition(":")
            if key.strip() == "Model name":
                model = val.strip()
            elif key.strip() == "Socket(s)":
                sockets = int(val.strip())
    except Exception:
        pass
    if model is None:
        try:
            with open("/proc/cpuinfo") as f:
                for ln in f:
                    if ln.startswith("model name"):
                        model = ln.partition(":")[2].strip()
                        break
        except Exception:
            pass
    return {"cpu_model": model, "sockets": sockets}

def oracle_rows_per_s(dist: str, seed: int, N: int, k: int, rows: list, threads: int, device="cpu"):
    """Time the oracle (as it stands) on a bounded sample of rows; returns rows/s.

    The sample rows are generated (bit-identically) on `device` and copied to
    the host; only the oracle call is timed."""
    import oracle
    import synth
    x = synth.row_subset(dist, seed, rows, N, device=device).cpu().numpy()
    oracle.build()
    t0 = time.perf_counter()
    oracle.select(x, k, nthreads=threads)
    dt = time.perf_counter() - t0
    return len(rows) / dt, dt


def select_config(Qr, N, k, dist, world):
    """The ksel_select workload config (shared by both arms)."""
    return {"workload": "ksel_select Q=%d N=%d k=%d %s" % (Qr, N, k, dist), "Q_per_rank": Qr,
            "Q_total": Qr * world, "N": N, "k": k, "dist": dist,
            "parallelism": "query-sharded x%d (no communication)" % world,
            "l2": "inputs (%.1f GiB/rank) far larger than L2; no flush" % (Qr * N * 4 / 2**30)}


def knn_config(N, Nl, Q, D, k, kind, mode, world):
    """The knn_search workload config (shared by both arms)."""
    return {"workload": "knn_search N=%d Q=%d D=%d k=%d %s (%s)" % (N, Q, D, k, kind, mode), "N": N,
            "N_per_rank": Nl, "Q": Q, "D": D, "k": k, "points": kind,
            "parallelism": ("reference rows sharded x%d + NCCL all-gather + ksel_merge" % world
                            if mode == "row-sharded" else "replicas x%d" % world),
            "l2": "reference image %.2f GB per rank (> L2)" % (Nl * D * 4 / 1e9)}


def run_reference_knn(args, rank, world):
    """--impl reference for the kNN configs: the oracle (double-precision triple
    loop + sort) on a bounded sample of queries per step."""
    if rank != 0:
        return
    import oracle
    import synth
    N, Q, D, k, kind, mode = KNN_CONFIGS[args.config]
    k = args.k or k
    threads = cpu_count()
    nref = N // world if mode == "row-sharded" else N
    ref = synth.knn_points(kind, 41, 0, nref, D).numpy()
    oracle.build()
    nq = max(4, threads)
    times = []
    for s in range(args.warmup + args.steps):
        qry = synth.knn_points(kind, 42, (s * nq) % Q, nq, D).numpy()
        t0 = time.perf_counter()
        oracle.knn(ref, qry, k, nthreads=threads)
        if s >= args.warmup:
            times.append(time.perf_counter() - t0)
    total = sum(times)
    value = nq * args.steps / total
    line = {
        "impl": "reference", "metric": "queries/sec (fused tcgen05 distance + k-selection)", "value": value,
        "unit": "queries/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * total / args.steps, "higher_is_better": True,
        "scaling": "strong" if mode == "row-sharded" else "weak", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "config": knn_config(N, nref, Q, D, k, kind, mode, world),
        "cpu_baseline": {"value": value, "unit": "queries/s", "cores": threads, "kind": "oracle",
                         "sample": "%d queries vs %d references per step" % (nq, nref), **cpu_info()},
        "e2e": {"value": value, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_reference(args, rank, world):
    if args.config in KNN_CONFIGS:
        return run_reference_knn(args, rank, world)
    Qr, N, k, dist = CONFIGS[args.config]
    k = args.k or k
    dist = args.dist or dist
    if rank != 0:
        return
    import synth
    threads = cpu_count()
    seed = synth.seed_for(3, dist)
    rows_per_step = max(4, 2 * threads)
    times = []
    q_all = Qr if args.scaling == "strong" else Qr * max(1, world)
    for s in range(args.warmup + args.steps):
        rows = [(s * rows_per_step + t) % q_all for t in range(rows_per_step)]
        _, dt = oracle_rows_per_s(dist, seed, N, k, rows, threads)
        if s >= args.warmup:
            times.append(dt)
    total = sum(times)
    value = rows_per_step * args.steps / total
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": select_config(Qr // world if args.scaling == "strong" else Qr, N, k, dist, world),
        "cpu_baseline": {"value": value, "unit": "rows/s", "cores": threads, "kind": "oracle",
                         "sample": "%d rows of N=%d per step (stable sort by (value,index), truncate to k)"
                                   % (rows_per_step, N), **cpu_info()},
        "e2e": {"value": value, "unit": "rows/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def timed_loop(args, step, world, rank, local_rank, dev, K, tdist):
    """Warm-up, a ~1 s clock soak, then EXACTLY args.steps timed steps between
    barriers + device syncs, CUDA events on the launching stream, max over ranks.
    Also returns the live CUDA-event time of the dominant kernel per launch."""
    import torch

    def barrier():
        if world > 1:
            tdist.barrier()

    stream = torch.cuda.current_stream(dev)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local_rank) if rank == 0 else None
    if sampler:
        sampler.start()
    t_soak = time.time()
    while time.time() - t_soak < 1.0:
        step()
        torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    K.timing_collect()  # drop anything recorded so far
    K.timing_enable(True)
    l0 = K.launch_count()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        step()
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    K.timing_enable(False)
    kern_ms, kern_n = K.timing_collect()
    launches = K.launch_count() - l0
    ms = ev0.elapsed_time(ev1)
    clocks = sampler.stop() if sampler else None
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    return float(t.item()), ms, kern_ms / max(1, kern_n), kern_n, launches, clocks


def bench_select(args, rank, world, local_rank, dev, K, tdist):
    import torch

    import synth

    Qr, N, k, dist = CONFIGS[args.config]
    k = args.k or k
    dist = args.dist or dist
    if args.scaling == "strong":  # configs[2]: Q rows in total, Q/g per rank
        row0, row1 = rank * Qr // world, (rank + 1) * Qr // world
        Qr = row1 - row0
    else:
        row0 = rank * Qr
    seed = synth.seed_for(3, dist)
    # ---- inputs resident in HBM (generation is not timed) ----------------------
    x = synth.rows(dist, seed, row0, Qr, N, device=dev)
    out_v = torch.empty((Qr, k), dtype=torch.float32, device=dev)
    out_i = torch.empty((Qr, k), dtype=torch.int32, device=dev)
    torch.cuda.synchronize()

    ms_max, ms_local, kern_ms, kern_n, launches, clocks = timed_loop(
        args, lambda: K.ksel_select(x, k, out_v, out_i), world, rank, local_rank, dev, K, tdist)
    ms_step = ms_max / args.steps
    rows_total = Qr * world
    value = rows_total / (ms_step / 1e3)
    # roofline of the dominant (only) kernel, timed live on the launching stream
    peak, peak_src = load_peaks()
    alg_bytes = Qr * (4.0 * N + 8.0 * k)
    # context for the denominator: a plain read-only stream over the same resident
    # input (torch's amax reduction, not our code), best of 3
    stream_gbs = None
    if rank == 0:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        best = None
        for _ in range(3):
            torch.cuda.synchronize()
            e0.record()
            torch.amax(x, dim=1)
            e1.record()
            torch.cuda.synchronize()
            t = e0.elapsed_time(e1)
            best = t if best is None else min(best, t)
        stream_gbs = Qr * N * 4.0 / (best / 1e3) / 1e9
    achieved = alg_bytes / (kern_ms / 1e3) / 1e9
    cfg = select_config(Qr, N, k, dist, world)
    workload = cfg["workload"]
    line = None
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
            "dtype": "f32", "data": "synthetic",
            "config": cfg,
            "hbm_gbs": achieved,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": load_traffic(workload), "peak_source": peak_src,
                         "kernel": "ksel_pool_kernel", "kernel_ms": kern_ms, "kernel_launches_timed": kern_n,
                         "bytes_per_launch": alg_bytes, "bytes_formula": "Q*(4N+8k)",
                         "read_stream_gbs": stream_gbs,
                         "read_stream_note": "torch.amax over the same resident input (context, not the peak)",
                         "peak_note": "the peak is a measured read+write copy; this kernel only reads (its "
                                      "writes are Q*k*8 bytes), so it can land slightly above 1.0 of it",
                         "nominal_gbs": 7700.0, "frac_nominal": achieved / 7700.0},
            "gpu_launches": launches,
            "clocks": clocks,
        }

    # ---- end-to-end through the public host API --------------------------------------
    if not args.no_e2e:
        er = min(args.e2e_rows or (2048 if world == 1 else 512), Qr)
        hx = torch.empty((er, N), dtype=torch.float32, pin_memory=True)
        hx.copy_(x[:er])
        hv = torch.empty((er, k), dtype=torch.float32, pin_memory=True)
        hi = torch.empty((er, k), dtype=torch.int32, pin_memory=True)
        ws = torch.empty(K.ksel_select_host_workspace(N, k), dtype=torch.uint8, device=dev)
        K.ksel_select_host(hx, k, hv, hi, workspace=ws, device=dev)
        if world > 1:
            tdist.barrier()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            K.ksel_select_host(hx, k, hv, hi, workspace=ws, device=dev)
        dt = torch.tensor([(time.perf_counter() - t0) / args.e2e_steps], dtype=torch.float64, device=dev)
        if world > 1:
            tdist.all_reduce(dt, op=tdist.ReduceOp.MAX)
        if rank == 0:
            line["e2e"] = {"value": er * world / float(dt.item()), "unit": "rows/s",
                           "h2d_bytes_per_step": er * N * 4, "d2h_bytes_per_step": er * k * 8,
                           "rows_per_step_per_rank": er, "api": "ksel_select_host (pinned host buffers)"}
        del hx, hv, hi, ws

    # ---- CPU baseline: the oracle on this host's cores (rank 0, N=1 only) --------
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        threads = cpu_count()
        # ~10-30 s of CPU work: 64 rows per host thread (first rows of each 2048-row block)
        nrows = args.cpu_sample_rows or min(Qr, 64 * threads)
        per_blk = max(1, nrows // max(1, Qr // 2048))
        sample = sorted({(b * 2048 + t) % Qr for b in range(max(1, Qr // 2048)) for t in range(per_blk)})[:nrows]
        rps, dt = oracle_rows_per_s(dist, seed, N, k, [row0 + r for r in sample], threads, device=dev)
        line["cpu_baseline"] = {"value": rps, "unit": "rows/s", "cores": threads, "kind": "oracle",
                                "sample": "%d rows of the same workload (%.1f s)" % (len(sample), dt),
                                **cpu_info()}
    return line


SWEEP_C2 = (1024, 65536, (1, 8, 32, 128, 256, 1024), ("U", "G", "DG", "SA", "SD", "T"))


def _kernel_ms(K, fn, reps):
    """Average device time of the dominant kernel of `fn` (the library's live CUDA
    events around each launch) and of the whole call (events around `reps`
    back-to-back calls on the current stream), after 3 warm-up calls."""
    import torch
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    K.timing_collect()
    K.timing_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    K.timing_enable(False)
    kms, kn = K.timing_collect()
    return kms / max(1, kn), e0.elapsed_time(e1) / reps


def run_sweep(dev, K, peak_hbm, peak_bf16):
    """The north star's k x distribution sweep (configs[1]) plus the kNN configs
    (configs[3] and configs[4]'s per-rank shape), one GPU, each entry's device
    time and roofline fraction.  Inputs (268 MB for C2, 512 MB of references for
    C4/C5) exceed the 126 MB L2 and are streamed anew by every call."""
    import torch

    import synth
    out = []
    Q, N, ks, dists = SWEEP_C2
    x = torch.empty((Q, N), dtype=torch.float32, device=dev)
    ov = torch.empty((Q, 1024), dtype=torch.float32, device=dev)
    oi = torch.empty((Q, 1024), dtype=torch.int32, device=dev)
    read_ms = None
    for dist in dists:
        synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, out=x)
        torch.cuda.synchronize()
        if read_ms is None:  # same-run read ceiling: torch row reductions over the same matrix (best)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            best = None
            for red in (lambda: torch.amin(x, dim=1), lambda: torch.amin(x), lambda: torch.sum(x, dim=1)):
                for _ in range(6):
                    e0.record()
                    red()
                    e1.record()
                    torch.cuda.synchronize()
                    t = e0.elapsed_time(e1)
                    best = t if best is None else min(best, t)
            read_ms = best
        for k in ks:
            v, i = ov[:, :k].contiguous(), oi[:, :k].contiguous()
            kms, cms = _kernel_ms(K, lambda: K.ksel_select(x, k, v, i), 20)
            gbs = Q * (4.0 * N + 8.0 * k) / (kms / 1e3) / 1e9
            out.append({"config": "c2", "op": "ksel_select", "Q": Q, "N": N, "k": k, "dist": dist,
                        "kernel": "ksel_pool_kernel", "ms": kms, "call_ms": cms, "rows_per_s": Q / (cms / 1e3),
                        "gbs": gbs, "frac_hbm": gbs / peak_hbm, "frac_read_ceiling": read_ms / kms})
    out.append({"config": "c2", "op": "read ceiling: best of torch.amin(x, dim=1), torch.amin(x), torch.sum(x, dim=1)",
                "Q": Q, "N": N, "ms": read_ms,
                "gbs": Q * N * 4.0 / (read_ms / 1e3) / 1e9})
    del x, ov, oi
    torch.cuda.empty_cache()
    for name, (Nr, Qk, D, k) in (("c4", (1000000, 10000, 128, 100)), ("c5-per-rank", (1000000, 10000, 128, 1024))):
        ref = synth.knn_points("knn-U", 41, 0, Nr, D, device=dev)
        qry = synth.knn_points("knn-U", 42, 0, Qk, D, device=dev)
        ws = torch.empty(K.knn_search_workspace(Nr, Qk, D, k), dtype=torch.uint8, device=dev)
        dv = torch.empty((Qk, k), dtype=torch.float32, device=dev)
        di = torch.empty((Qk, k), dtype=torch.int32, device=dev)
        kms, cms = _kernel_ms(K, lambda: K.knn_search(ref, qry, k, out_dist=dv, out_idx=di, workspace=ws), 5)
        tf = 2.0 * Qk * Nr * D / (kms / 1e3) / 1e12
        tf_call = 2.0 * Qk * Nr * D / (cms / 1e3) / 1e12
        out.append({"config": name, "op": "knn_search", "N": Nr, "Q": Qk, "D": D, "k": k, "points": "knn-U",
                    "kernel": "knn_fused_kernel", "ms": kms, "call_ms": cms, "queries_per_s": Qk / (cms / 1e3),
                    "tflops": tf, "frac_tensor": tf / peak_bf16, "frac_tensor_call": tf_call / peak_bf16,
                    "flops_formula": "2*Q*N*D (algorithmic, one pass)"})
        del ref, qry, ws, dv, di
        torch.cuda.empty_cache()
    return out


def run_knn_row_sharded(args, rank, world, dev, K, tdist):
    """configs[4] over the process group: N = 8*10^6 references sharded by rows (10^6 per
    rank at g = 8; N = 10^6 * g in total for g < 8 so every rank keeps the per-rank shape),
    Q = 10^4, k = 1024, each rank's search writing into the chunked all-gather buffers and
    merging its query slices in place (dist.knn_search_sharded; NCCL over NVLink).  Device
    time between barriers, max over ranks; bit-exactness of this path is tested in
    tests/test_dist_gpu.py (same function, real kernels)."""
    import torch

    import synth
    from paper_conf_ipps_tang0emg15_b200 import dist as kd
    N = 1000000 * world if world < 8 else 8000000
    Q, D, k = 10000, 128, 1024
    r0, r1 = kd.shard_range(N, world, rank)
    ref = synth.knn_points("knn-U", 41, r0, r1 - r0, D, device=dev)
    qry = synth.knn_points("knn-U", 42, 0, Q, D, device=dev)
    ws = torch.empty(K.knn_search_workspace(r1 - r0, Q, D, k), dtype=torch.uint8, device=dev)

    def local_knn(rs, qq, kk, off, out_v, out_i):
        K.knn_search(rs, qq, kk, idx_offset=off, out_dist=out_v, out_idx=out_i, workspace=ws)

    chunks = int(os.environ.get("KSEL_BENCH_CHUNKS", "0")) or kd.auto_chunks(Q)

    def step():
        return kd.knn_search_sharded(ref, qry, k, N, local_knn=local_knn, chunks=chunks)

    for _ in range(2):
        step()
    torch.cuda.synchronize()
    steps = 3
    if world > 1:
        tdist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        v, i, qids = step()
    e1.record()
    torch.cuda.synchronize()
    t = torch.tensor([e0.elapsed_time(e1) / steps], dtype=torch.float64, device=dev)
    if world > 1:
        tdist.barrier()
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    ms = float(t.item())
    # every query merged by exactly one rank, k ascending distances each
    nq = torch.tensor([qids.numel()], dtype=torch.int64, device=dev)
    if world > 1:
        tdist.all_reduce(nq)
    ok = int(nq.item()) == Q and bool((v[:, 1:] >= v[:, :-1]).all().item())
    del ref, qry, ws
    torch.cuda.empty_cache()
    return {"workload": "knn_search N=%d (row-sharded x%d) Q=%d D=%d k=%d knn-U" % (N, world, Q, D, k),
            "ms_per_step": ms, "queries_per_s": Q / (ms / 1e3), "chunks": chunks,
            "exchange": "async all_gather_into_tensor per query chunk (%s) + in-place merge; chunks: "
                        "dist.auto_chunks (1 at Q = 10^4: chunking the search costs more than the "
                        "exchange it hides, profiles/r02_knn_sharded_chunks.txt)" % ("NCCL" if world > 1 else "single rank"),
            "tflops_per_rank": 2.0 * Q * (r1 - r0) * D / (ms / 1e3) / 1e12, "queries_covered_sorted": ok}


KNN_CONFIGS = {
    # name: (N total, Q, D, k, point kind, mode)
    "c4": (1000000, 10000, 128, 100, "knn-U", "replica"),
    "c5": (8000000, 10000, 128, 1024, "knn-U", "row-sharded"),
}


def bench_knn(args, rank, world, local_rank, dev, K, tdist):
    import torch

    import synth
    from paper_conf_ipps_tang0emg15_b200 import dist as kd

    N, Q, D, k, kind, mode = KNN_CONFIGS[args.config]
    k = args.k or k
    kind = args.dist or kind
    if mode == "row-sharded":
        r0, r1 = kd.shard_range(N, world, rank)
    else:
        r0, r1 = 0, N
    Nl = r1 - r0
    ref = synth.knn_points(kind, 41, r0, Nl, D, device=dev)
    qry = synth.knn_points(kind, 42, 0, Q, D, device=dev)
    ws = torch.empty(K.knn_search_workspace(Nl, Q, D, k), dtype=torch.uint8, device=dev)
    ov = torch.empty((Q, k), dtype=torch.float32, device=dev)
    oi = torch.empty((Q, k), dtype=torch.int32, device=dev)
    torch.cuda.synchronize()

    if mode == "row-sharded" and world > 1:
        def local_knn(rs, qq, kk, off, out_v, out_i):
            K.knn_search(rs, qq, kk, idx_offset=off, out_dist=out_v, out_idx=out_i, workspace=ws)

        def step():
            return kd.knn_search_sharded(ref, qry, k, N, local_knn=local_knn)
    else:
        def step():
            return K.knn_search(ref, qry, k, idx_offset=r0, out_dist=ov, out_idx=oi, workspace=ws)

    ms_max, ms_local, kern_ms, kern_n, launches, clocks = timed_loop(args, step, world, rank, local_rank, dev, K, tdist)
    ms_step = ms_max / args.steps
    q_total = Q if mode == "row-sharded" else Q * world
    value = q_total / (ms_step / 1e3)
    peaks_bf16, src = 1637.7, "measured (MEASURED_PEAKS.json bf16_tflops, burst)"
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            peaks_bf16 = float(json.load(f)["bf16_tflops"])
    except Exception:
        src = "fallback (B200_PROFILING.md 1.59 PFLOP/s)"
        peaks_bf16 = 1590.0
    flops = 2.0 * Q * Nl * D  # algorithmic single-pass dot products of this rank's launch
    achieved = flops / (kern_ms / 1e3) / 1e12
    cfg = knn_config(N, Nl, Q, D, k, kind, mode, world)
    workload = cfg["workload"]
    line = None
    if rank == 0:
        line = {
            "metric": "queries/sec (fused tcgen05 distance + k-selection)", "value": value, "unit": "queries/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "strong" if mode == "row-sharded" else "weak",
            "vs_baseline": None, "dtype": "fp16 filter (centred, per-tile power-of-two scales, fp32 acc) + f64 exact rescoring", "data": "synthetic",
            "config": cfg,
            "roofline": {"bound": "tensor", "achieved": achieved, "peak": peaks_bf16, "unit": "TFLOP/s",
                         "frac": achieved / peaks_bf16, "traffic": load_traffic(workload), "peak_source": src,
                         "kernel": "knn_fused_kernel", "kernel_ms": kern_ms,
                         "flops_per_launch": flops, "flops_formula": "2*Q*N_rank*D (algorithmic, 1 pass; "
                                                                     "executed: 1 fp16 pass + a bf16 norm block; the speculative pre-pass launch over up to 128 sampled tiles is counted in the call, not in this kernel)",
                         "note": "kernel = the fused filter; the call adds the prologue and the exact "
                                 "rescoring (bit-identical to the oracle)"},
            "gpu_launches": launches,
            "clocks": clocks,
        }
    if not args.no_e2e:
        # end to end: pinned host inputs copied in every step, results copied back
        href = torch.empty((Nl, D), dtype=torch.float32, pin_memory=True)
        href.copy_(ref)
        hq = torch.empty((Q, D), dtype=torch.float32, pin_memory=True)
        hq.copy_(qry)
        hv = torch.empty((Q, k), dtype=torch.float32, pin_memory=True)
        hi = torch.empty((Q, k), dtype=torch.int32, pin_memory=True)

        # Every step copies its inputs host -> device and its result back; the copy of
        # step s+1's inputs (on a copy stream, into the other of two device buffers)
        # overlaps step s's kernels -- the double buffering ksel_select_host does inside.
        cur = torch.cuda.current_stream(dev)
        cps = torch.cuda.Stream(device=dev)
        refb = [ref, torch.empty_like(ref)]
        qryb = [qry, torch.empty_like(qry)]
        landed = [torch.cuda.Event(), torch.cuda.Event()]
        used = [torch.cuda.Event(), torch.cuda.Event()]

        def issue_copy(b):
            with torch.cuda.stream(cps):
                cps.wait_event(used[b])  # the step that last read buffer b is done
                refb[b].copy_(href, non_blocking=True)
                qryb[b].copy_(hq, non_blocking=True)
                landed[b].record(cps)

        def e2e_run(steps):
            for b in (0, 1):
                used[b].record(cur)
            issue_copy(0)
            for s_ in range(steps):
                b = s_ & 1
                if s_ + 1 < steps:
                    issue_copy(b ^ 1)
                cur.wait_event(landed[b])
                v, i = K.knn_search(refb[b], qryb[b], k, idx_offset=r0, out_dist=ov, out_idx=oi, workspace=ws)
                used[b].record(cur)
                hv.copy_(v, non_blocking=True)
                hi.copy_(i, non_blocking=True)
            torch.cuda.synchronize()

        e2e_run(2)
        nst = max(args.e2e_steps, 8)  # (the first copy is not overlapped: amortise it over 8 steps)
        t0 = time.perf_counter()
        e2e_run(nst)
        dt = torch.tensor([(time.perf_counter() - t0) / nst], dtype=torch.float64, device=dev)
        if world > 1:
            tdist.all_reduce(dt, op=tdist.ReduceOp.MAX)
        if rank == 0:
            line["e2e"] = {"value": q_total / float(dt.item()), "unit": "queries/s",
                           "h2d_bytes_per_step": (Nl + Q) * D * 4, "d2h_bytes_per_step": Q * k * 8,
                           "api": "knn_search; each step's pinned host inputs copied in (the copy for step "
                                  "s+1 overlapping step s, double-buffered) and its result copied back"
                                  + ("; per-shard search, cross-rank merge not included"
                                     if mode == "row-sharded" and world > 1 else "")}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        threads = cpu_count()
        nq = max(8, 2 * threads)
        hr = ref.cpu().numpy()
        hq = qry[:nq].cpu().numpy()
        oracle.build()
        t0 = time.perf_counter()
        oracle.knn(hr, hq, k, nthreads=threads)
        dt = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": nq / dt, "unit": "queries/s", "cores": threads, "kind": "oracle",
                                "sample": "%d queries vs all %d references (%.1f s)" % (nq, Nl, dt), **cpu_info()}
    return line


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as tdist

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        tdist.init_process_group("nccl", device_id=dev)
    elif args.knn_sharded == "on":  # single-rank NCCL group: exercises the sharded path on one GPU
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        tdist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)

    import paper_conf_ipps_tang0emg15_b200 as K

    if args.config in KNN_CONFIGS:
        line = bench_knn(args, rank, world, local_rank, dev, K, tdist)
    else:
        line = bench_select(args, rank, world, local_rank, dev, K, tdist)
        if rank == 0 and world == 1 and not args.no_sweep and args.config == "c3":
            import torch
            torch.cuda.empty_cache()
            peak_bf16 = 1646.1
            try:
                with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
                    peak_bf16 = float(json.load(f)["bf16_tflops"])
            except Exception:
                pass
            line["sweep"] = run_sweep(dev, K, line["roofline"]["peak"], peak_bf16)
        if args.config == "c3" and (args.knn_sharded == "on" or (args.knn_sharded == "auto" and world > 1)):
            import torch
            torch.cuda.empty_cache()
            ks = run_knn_row_sharded(args, rank, world, dev, K, tdist)
            if rank == 0:
                line["knn_row_sharded"] = ks
    if rank == 0:
        print(json.dumps(line), flush=True)
    if tdist.is_initialized():
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
