#!/usr/bin/env python
"""bench.py -- batched k-selection throughput on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...

Workload (BASELINE.json configs[2], the 1/2/4/8-GPU config): ksel_select over
Q = 16384 rows per GPU of N = 2^20 uniform fp32 distances, k = 256,
query-sharded (rank r owns global rows [r*Q, (r+1)*Q); no communication;
weak scaling).  A step is one ksel_select call over the rank's rows, inputs
resident in HBM (64 GiB per GPU, far larger than the 126 MB L2, so no flush is
needed between steps).  Metric: selected rows/s (whole job) and achieved HBM
GB/s vs the measured peak.

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
    ap.add_argument("--config", choices=sorted(CONFIGS), default="c3")
    ap.add_argument("--k", type=int, default=None)
    ap.add_argument("--dist", default=None)
    ap.add_argument("--scaling", choices=["weak", "strong"], default="weak")
    ap.add_argument("--e2e-rows", type=int, default=2048, help="rows per end-to-end step (host buffers)")
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


def run_reference(args, rank, world):
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
    for s in range(args.warmup + args.steps):
        rows = [(s * rows_per_step + t) % (Qr * max(1, world)) for t in range(rows_per_step)]
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
        "config": {"workload": "ksel_select Q=%d/rank N=%d k=%d %s (oracle on host cores)" % (Qr, N, k, dist),
                   "Q_per_rank": Qr, "N": N, "k": k, "dist": dist},
        "cpu_baseline": {"value": value, "unit": "rows/s", "cores": threads, "kind": "oracle",
                         "sample": "%d rows of N=%d per step (stable sort by (value,index), truncate to k)"
                                   % (rows_per_step, N)},
        "e2e": {"value": value, "unit": "rows/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


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

    import paper_conf_ipps_tang0emg15_b200 as K
    import synth

    Qr, N, k, dist = CONFIGS[args.config]
    k = args.k or k
    dist = args.dist or dist
    Qglob = Qr * world
    if args.scaling == "strong":
        Qglob = Qr
        Qr = Qglob // world
    row0 = rank * Qr
    seed = synth.seed_for(3, dist)

    # ---- inputs resident in HBM (generation is not timed) ----------------------
    x = synth.rows(dist, seed, row0, Qr, N, device=dev)
    out_v = torch.empty((Qr, k), dtype=torch.float32, device=dev)
    out_i = torch.empty((Qr, k), dtype=torch.int32, device=dev)
    torch.cuda.synchronize()

    def barrier():
        if world > 1:
            tdist.barrier()

    stream = torch.cuda.current_stream(dev)
    for _ in range(args.warmup):
        K.ksel_select(x, k, out_v, out_i)
    torch.cuda.synchronize()

    # clocks: sample during a ~1 s soak of the same step and the timed region
    sampler = ClockSampler(local_rank) if rank == 0 else None
    if sampler:
        sampler.start()
    t_soak = time.time()
    while time.time() - t_soak < 1.0:
        K.ksel_select(x, k, out_v, out_i)
        torch.cuda.synchronize()

    barrier()
    torch.cuda.synchronize()
    l0 = K.launch_count()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        K.ksel_select(x, k, out_v, out_i)
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    launches = K.launch_count() - l0
    ms = ev0.elapsed_time(ev1)
    clocks = sampler.stop() if sampler else None

    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    ms_max = float(t.item())
    ms_step = ms_max / args.steps
    rows_total = Qr * world
    value = rows_total / (ms_step / 1e3)

    # roofline of the dominant (only) kernel: one launch per step on this stream
    peak, peak_src = load_peaks()
    alg_bytes = Qr * (4.0 * N + 8.0 * k)
    achieved = alg_bytes / (ms / args.steps / 1e3) / 1e9
    workload = "ksel_select Q=%d N=%d k=%d %s" % (Qr, N, k, dist)
    traffic = load_traffic(workload)

    line = None
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "rows/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
            "dtype": "f32", "data": "synthetic",
            "config": {"workload": workload, "Q_per_rank": Qr, "Q_total": rows_total, "N": N, "k": k,
                       "dist": dist, "parallelism": "query-sharded x%d (no communication)" % world,
                       "l2": "inputs (%.1f GiB/rank) far larger than L2; no flush" % (Qr * N * 4 / 2**30)},
            "hbm_gbs": achieved,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                         "kernel": "ksel_pool_kernel",
                         "bytes_per_launch": alg_bytes, "bytes_formula": "Q*(4N+8k)"},
            "gpu_launches": launches,
            "clocks": clocks,
        }

    # ---- end-to-end through the public host API (rank 0 .. all ranks) -------------
    if not args.no_e2e:
        er = min(args.e2e_rows, Qr)
        hx = torch.empty((er, N), dtype=torch.float32, pin_memory=True)
        hx.copy_(x[:er])
        hv = torch.empty((er, k), dtype=torch.float32, pin_memory=True)
        hi = torch.empty((er, k), dtype=torch.int32, pin_memory=True)
        ws = torch.empty(K.ksel_select_host_workspace(N, k), dtype=torch.uint8, device=dev)
        K.ksel_select_host(hx, k, hv, hi, workspace=ws, device=dev)
        barrier()
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
                                "sample": "%d rows of the same workload (%.1f s)" % (len(sample), dt)}

    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
