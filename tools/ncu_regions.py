"""Attribute executed instructions of the pool kernel to algorithm phases.

Every SASS instruction of an ncu source-page CSV (cuda,sass) gets its own source
line; instructions from headers (inlined helpers) take the phase of the nearest
preceding select_pool.cu instruction by address.  __noinline__ functions are their
own phase.  usage: python tools/ncu_regions.py <src.csv>"""
import csv
import sys

REGIONS = [  # select_pool.cu line ranges -> phase
    (113, 219, "setup/order"), (220, 302, "exact-path"), (303, 319, "head-tail"),
    (320, 377, "start-bound"), (378, 436, "stream+filter"), (437, 470, "final"), (470, 600, "other")]


def region(line):
    for a, b, n in REGIONS:
        if a <= line < b:
            return n
    return "other"


rows = []
fname, func = "?", "?"
for r in csv.reader(open(sys.argv[1])):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        func = r[1]
        continue
    if r[0] == "Line No":
        continue
    if r[0] != "":
        cur_line = int(r[0]) if r[0].isdigit() else -1
        continue
    # SASS row: "", "", address, sass, ..., instructions executed at index 7
    try:
        addr = int(r[2], 16)
        ex = int(r[7])
    except (ValueError, IndexError):
        continue
    rows.append((func, addr, fname, cur_line, ex, r[3].strip()))
tot = {}
allx = sum(x[4] for x in rows) or 1
for func in sorted(set(x[0] for x in rows)):
    fr = sorted((x for x in rows if x[0] == func), key=lambda x: x[1])
    short = func.split("(")[0].split("::")[-1][:40]
    last = None
    for _, addr, fn, line, ex, sass in fr:
        if "ksel_pool_kernel" not in short:
            ph = "fn:" + short
        elif fn == "select_pool.cu":
            ph = region(line)
            last = ph
        else:
            ph = last or "setup/order"
        tot[ph] = tot.get(ph, 0) + ex
print("total warp instructions %d" % allx)
for ph, ex in sorted(tot.items(), key=lambda x: -x[1]):
    print("%-40s %12d  %5.1f%%" % (ph, ex, 100.0 * ex / allx))
