"""A/B timing of ksel_select between libksel_A.so (tools/ab_build.sh) and libksel.so in
one GPU session: the two libraries alternate in fresh processes, rounds x configs.
usage: python tools/ab_select.py "Q,N,k,dist;..." [rounds]"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, torch
sys.path.insert(0, sys.argv[1])
import paper_conf_ipps_tang0emg15_b200 as K, synth
for cfg in sys.argv[2].split(";"):
    Q, N, k, dist = cfg.split(","); Q, N, k = int(Q), int(N), int(k)
    x = synth.rows(dist, synth.seed_for(2, dist), 0, Q, N, device="cuda")
    for _ in range(3): K.ksel_select(x, k)
    torch.cuda.synchronize(); K.timing_collect(); K.timing_enable(True)
    reps = max(3, min(20, int(2e9 / (Q * N * 4))))
    for _ in range(reps): K.ksel_select(x, k)
    torch.cuda.synchronize(); K.timing_enable(False)
    ms, n = K.timing_collect()
    print("%s %.4f" % (cfg, ms / n), flush=True)
    del x; torch.cuda.empty_cache()
"""
cfgs = sys.argv[1]
rounds = int(sys.argv[2]) if len(sys.argv) > 2 else 3
res = {}
for r in range(rounds):
    for lib in ("libksel_A.so", "libksel.so"):
        env = dict(os.environ, KSEL_AB_LIB=lib)
        out = subprocess.run([sys.executable, "-c", CHILD, ROOT, cfgs], env=env, capture_output=True, text=True,
                             timeout=900)
        if out.returncode:
            print(out.stderr[-1500:])
        for ln in out.stdout.split("\n"):
            if ln.strip():
                cfg, ms = ln.rsplit(" ", 1)
                res.setdefault(cfg, {}).setdefault(lib, []).append(float(ms))
print("%-28s %10s %10s %7s" % ("config", "A (min)", "B (min)", "B/A"))
for cfg, d in res.items():
    a, b = min(d.get("libksel_A.so", [float("nan")])), min(d.get("libksel.so", [float("nan")]))
    print("%-28s %10.4f %10.4f %7.3f" % (cfg, a, b, b / a))
