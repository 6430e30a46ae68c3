"""Per-CUDA-source-line instruction and stall totals from an ncu report (cuda,sass view).

    python tools/ncu_src_lines.py <report.ncu-rep> [top_n]
"""
import csv
import subprocess
import sys

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
fname, res = "?", []
for r in csv.reader(out.splitlines()):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] in ("Function Name", "Line No") or r[0] == "":
        continue
    try:
        st, ex = int(r[4]), int(r[7])
    except (ValueError, IndexError):
        continue
    res.append((ex, st, "%s:%s" % (fname, r[0]), r[1].strip()[:90]))
tex = sum(x[0] for x in res) or 1
tst = sum(x[1] for x in res) or 1
print("instructions %d  stall samples %d" % (tex, tst))
for ex, st, loc, src in sorted(res, reverse=True)[:n]:
    print("%5.1f%% ex %5.1f%% st  %-22s %s" % (100.0 * ex / tex, 100.0 * st / tst, loc, src))
