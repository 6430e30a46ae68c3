"""Build libksel.so (the C-ABI CUDA library) in-tree for sm_100a with nvcc.

The .so lands next to this file so it travels with the repo snapshot to the
GPU box (it is git-ignored, not gpurun-ignored).  Objects are compiled in
parallel and cached under build/ by source hash.
"""
from __future__ import annotations

import concurrent.futures as cf
import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libksel.so")
OBJDIR = os.path.join(ROOT, "build", "obj")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

NVCC_FLAGS = [
    "-std=c++17", "-O3", "-lineinfo",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
    "--expt-relaxed-constexpr",
    "-Xptxas", "-warn-spills",
    "-I" + INCLUDE, "-I" + CSRC,
]
# Timing-experiment kernel variants (pipeline-only / counter modes, 1-pass MMA, other
# epilogue shapes) are compiled only into an experiments build; the product library
# (the default) contains none of them and reads no result-affecting knob.
if os.environ.get("KSEL_BUILD_EXPERIMENTS") == "1":
    NVCC_FLAGS.append("-DKSEL_EXPERIMENTS")
    LIB = os.path.join(HERE, "libksel_exp.so")  # never the product library


def _sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cu"))


def _headers():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".cuh", ".h"))]
    hs += [os.path.join(INCLUDE, f) for f in os.listdir(INCLUDE) if f.endswith(".h")]
    return sorted(hs)


SPLIT_R = (1, 2, 4, 8, 16, 32)  # queue sizes k' = 32*R; "// KSEL_SPLIT_R" sources build once per R


def _digest(src: str, extra: list) -> str:
    h = hashlib.sha256()
    for p in [src] + _headers():
        with open(p, "rb") as f:
            h.update(f.read())
    h.update(" ".join(NVCC_FLAGS + extra).encode())
    return h.hexdigest()[:16]


def _units():
    """(source, extra flags, object tag) for every compilation unit."""
    units = []
    for src in _sources():
        with open(src) as f:
            first = f.readline()
        if "KSEL_SPLIT_R" in first:
            units += [(src, ["-DKSEL_ONLY_R=%d" % r], "r%d" % r) for r in SPLIT_R]
        else:
            units.append((src, [], "all"))
    return units


def _compile(unit, verbose: bool) -> str:
    src, extra, tag = unit
    os.makedirs(OBJDIR, exist_ok=True)
    obj = os.path.join(OBJDIR, "%s.%s.%s.o" % (os.path.basename(src), tag, _digest(src, extra)))
    if os.path.exists(obj):
        return obj
    cmd = [NVCC] + NVCC_FLAGS + extra + ["-c", src, "-o", obj + ".tmp"]
    if verbose:
        print(" ".join(cmd), flush=True)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, r.stdout, r.stderr))
    if r.stderr.strip() and verbose:
        print(r.stderr, file=sys.stderr)
    os.replace(obj + ".tmp", obj)
    return obj


def build(verbose: bool = False) -> str:
    """Compile every csrc/*.cu for sm_100a and link libksel.so; returns its path."""
    units = _units()
    workers = int(os.environ.get("KSEL_BUILD_JOBS", str(max(2, os.cpu_count() or 2))))
    with cf.ThreadPoolExecutor(max_workers=min(workers, len(units))) as ex:
        objs = list(ex.map(lambda u: _compile(u, verbose), units))
    for f in os.listdir(OBJDIR):  # drop stale objects of older sources
        if os.path.join(OBJDIR, f) not in objs and f.endswith(".o"):
            os.remove(os.path.join(OBJDIR, f))
    stamp = hashlib.sha256("|".join(objs).encode()).hexdigest()[:16]
    stamp_file = LIB + ".stamp"
    if os.path.exists(LIB) and os.path.exists(stamp_file) and open(stamp_file).read() == stamp:
        return LIB
    cmd = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", LIB + ".tmp"] + objs + ["-lcudart"]
    if verbose:
        print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    with open(stamp_file, "w") as f:
        f.write(stamp)
    return LIB


if __name__ == "__main__":
    print(build(verbose=True))
