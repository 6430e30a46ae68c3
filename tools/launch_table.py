"""Summarise an ncu --metrics gpu__time_duration.sum launch list: per kernel count and mean time."""
import collections
import csv
import sys

agg = collections.OrderedDict()
hdr = None
for r in csv.reader(open(sys.argv[1])):
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            scale = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(d.get("Metric Unit", "nsecond"), 1e-3)
            agg.setdefault(d["Kernel Name"].split("(")[0], []).append(float(d["Metric Value"].replace(",", "")) * scale)
tot = sum(sum(v) for v in agg.values())
for k, v in agg.items():
    print("%-48s n=%3d mean=%9.1f us  share=%5.1f%%" % (k[:48], len(v), sum(v) / len(v), 100 * sum(v) / tot))
