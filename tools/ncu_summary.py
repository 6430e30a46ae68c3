"""Summarise an ncu report (raw page): key throughput metrics and stall reasons.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--json out.json]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed.avg.per_cycle_active", "smsp__inst_executed.sum", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "launch__occupancy_limit_shared_mem",
    "launch__shared_mem_per_block_dynamic", "launch__waves_per_multiprocessor",
    "sm__cycles_elapsed.avg.per_second", "lts__t_bytes.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "smsp__inst_executed_op_shfl.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
]


def load(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2:]
    return hdr, units, vals


def main():
    path = sys.argv[1]
    hdr, units, vals = load(path)
    res = []
    for v in vals:
        d = {"kernel": v[hdr.index("Kernel Name")] if "Kernel Name" in hdr else ""}
        for k in KEYS:
            if k in hdr:
                d[k] = v[hdr.index(k)] + " " + units[hdr.index(k)]
        stalls = {}
        for i, n in enumerate(hdr):
            if n.startswith("smsp__pcsamp_warps_issue_stalled_") and not n.endswith("_not_issued"):
                try:
                    c = float(v[i])
                except ValueError:
                    continue
                if c > 0:
                    stalls[n.replace("smsp__pcsamp_warps_issue_stalled_", "")] = c
        tot = sum(stalls.values()) or 1
        d["stall_pct"] = {k: round(100 * c / tot, 1) for k, c in sorted(stalls.items(), key=lambda x: -x[1])[:10]}
        res.append(d)
    txt = json.dumps(res, indent=1)
    if "--json" in sys.argv:
        with open(sys.argv[sys.argv.index("--json") + 1], "w") as f:
            f.write(txt + "\n")
    print(txt)


if __name__ == "__main__":
    main()
