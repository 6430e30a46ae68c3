"""C2 (Q=1024, N=65536) ksel_pool_kernel phase costs: kernel time with phases switched
off (KSEL_POOL_SKIP bits of the -DKSEL_EXPERIMENTS build: 8 = no exact admission path,
16 = no final select/sort/merge, 32 = no starting bound; results are wrong in those
modes, only the time is of interest).  usage: python tools/c2_phases.py [dists] [ks]"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_ipps_tang0emg15_b200 as K, synth
Q, N = 1024, 65536
x = torch.empty((Q, N), dtype=torch.float32, device="cuda")
for dist in sys.argv[2].split(","):
    synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, out=x)
    for k in [int(v) for v in sys.argv[3].split(",")]:
        for _ in range(3):
            K.ksel_select(x, k)
        torch.cuda.synchronize()
        K.timing_collect(); K.timing_enable(True)
        for _ in range(20):
            K.ksel_select(x, k)
        torch.cuda.synchronize(); K.timing_enable(False)
        ms, n = K.timing_collect()
        print("%s k=%d %.4f" % (dist, k, ms / n), flush=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
best = 1e9
for _ in range(6):
    e0.record(); torch.amin(x); e1.record(); torch.cuda.synchronize(); best = min(best, e0.elapsed_time(e1))
print("amin %.4f" % best)
"""
dists = sys.argv[1] if len(sys.argv) > 1 else "U,T,SD"
ks = sys.argv[2] if len(sys.argv) > 2 else "8,256,1024"
exp = os.environ.get("C2_EXP", "1") == "1"
modes = [int(m) for m in os.environ.get("C2_MODES", "0,8,16,32,56").split(",")] if exp else [0]
res = {}
for m in modes:
    env = dict(os.environ, KSEL_POOL_SKIP=str(m))
    if exp:
        env["KSEL_EXPERIMENTS_LIB"] = "1"
    out = subprocess.run([sys.executable, "-c", CHILD, ROOT, dists, ks], env=env, capture_output=True,
                         text=True, timeout=600)
    if out.returncode:
        print(out.stderr[-2000:])
    for ln in out.stdout.split("\n"):
        if ln.strip():
            key, val = ln.rsplit(" ", 1)
            res.setdefault(key, {})[m] = float(val)
hdr = "%-14s" % "case" + "".join("%10s" % ("skip=%d" % m) for m in modes)
print(hdr)
for key, row in res.items():
    print("%-14s" % key + "".join("%10.4f" % row.get(m, float("nan")) for m in modes))
