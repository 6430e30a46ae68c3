"""Top SASS instructions by stall samples / executions from an ncu report (source page)."""
import csv
import subprocess
import sys

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
data = rows[2:]
ia, isrc = hdr.index("Address"), hdr.index("Source")
iexe, ist = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
num = lambda r, i: int(r[i]) if r[i].isdigit() else 0
tot_st = sum(num(r, ist) for r in data)
tot_ex = sum(num(r, iexe) for r in data)
print("instructions %d  stall samples %d" % (tot_ex, tot_st))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
# windows of 16 instructions: where do stalls concentrate?
win = 16
agg = []
for i in range(0, len(data), win):
    blk = data[i:i + win]
    agg.append((sum(num(r, ist) for r in blk), sum(num(r, iexe) for r in blk), blk[0][ia][-5:],
                " | ".join(r[isrc].strip()[:28] for r in blk if num(r, ist) > 0.002 * tot_st)[:160]))
for st, ex, a, txt in sorted(agg, reverse=True)[:n]:
    print("%5.1f%% st  %5.1f%% ex  %s  %s" % (100.0 * st / tot_st, 100.0 * ex / max(tot_ex, 1), a, txt))
