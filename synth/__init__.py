"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This module holds NONE of the method's arithmetic: it only produces input bits.
Every value is a pure function of (seed, global row, column) through a 32-bit
counter-based integer hash evaluated with exact torch int64 ops, so

* the same row has identical bits on CPU and on any GPU (integer ops are exact,
  the int->float conversions and the few fp32 adds/multiplies below are single
  IEEE operations evaluated the same way on every device);
* a row does not depend on how rows are blocked or sharded across ranks
  (query sharding) -- rank r can generate rows [a, b) alone and
  the oracle can regenerate any sampled row on the host.

Distributions (SURVEY.md 8(d) "Synthetic inputs"; paper workload PAPER.md L243:
"randomly generated ... each value distributed in the range of [0, 1]" and
"we can assume the k-NNs are randomly distributed in each list"):

  U   uniform [0,1) with 24-bit resolution
  G   Gaussian-shaped (Irwin-Hall of 4 uniforms, mean 0, var 1)
  DG  distance-shaped 21.33 + 2.23*G: the squared L2 between uniform [0,1]^128
      points (mean 128/6, sd ~2.2), i.e. the rows k-selection sees in the
      paper's k-NN workload; all values share one fp32 exponent
  SA  per-row sorted ascending (best case: exactly k admits)
  SD  per-row sorted descending (worst case for an in-order threshold)
  T   heavy ties: 16 distinct integer values
  X   special values: +-0.0, +-Inf, NaN, +-denormal mixed with U

k-NN points: ``knn-U`` uniform [0,1)^D and ``knn-S``
SIFT-shaped non-negative integers in [0,255] (skewed towards 0).
"""
from __future__ import annotations

import torch

M32 = 0xFFFFFFFF
DISTS = ("U", "G", "DG", "SA", "SD", "T", "X")
_TAG = {"U": 1, "G": 2, "DG": 3, "SA": 4, "SD": 5, "T": 6, "X": 7, "knn-U": 8, "knn-S": 9}
_CHUNK = 1 << 24  # elements per generation chunk (bounds int64 temporaries)


def seed_for(config: int, dist: str, block: int = 0) -> int:
    """seed = 1000*config + 10*distribution + block."""
    return 1000 * config + 10 * _TAG[dist] + block


def _mix32(x: torch.Tensor) -> torch.Tensor:
    # lowbias32-style avalanche on values in [0, 2^32); both multipliers are
    # < 2^31 so every product fits in int64 without overflow.
    x = x ^ (x >> 16)
    x = (x * 0x7FEB352D) & M32
    x = x ^ (x >> 15)
    x = (x * 0x2C1B3C6D) & M32
    x = x ^ (x >> 16)
    return x


def _hash(seed: int, tag: int, rows: torch.Tensor, cols: torch.Tensor, stream: int) -> torch.Tensor:
    """32-bit hash of (seed, tag, row, col, stream); rows [R,1], cols [1,C] int64."""
    base = ((seed * 0x9E3779B1) ^ (tag << 24) ^ (stream * 0x85EBCA6B)) & M32
    hr = _mix32((rows * 0x61C88647 + base) & M32)
    return _mix32(hr ^ _mix32(cols & M32))


def _u24(h: torch.Tensor) -> torch.Tensor:
    return (h >> 8).to(torch.float32) * (1.0 / 16777216.0)


def _gen_block(dist: str, seed: int, rows: torch.Tensor, N: int, device) -> torch.Tensor:
    cols = torch.arange(N, device=device, dtype=torch.int64).unsqueeze(0)
    tag = _TAG[dist]
    if dist in ("U", "SA", "SD"):
        out = _u24(_hash(seed, tag, rows, cols, 0))
        if dist == "SA":
            out = torch.sort(out, dim=1).values
        elif dist == "SD":
            out = torch.flip(torch.sort(out, dim=1).values, dims=[1])
        return out
    if dist in ("G", "DG"):
        s = _u24(_hash(seed, tag, rows, cols, 0))
        for st in (1, 2, 3):
            s = s + _u24(_hash(seed, tag, rows, cols, st))
        g = (s - 2.0) * 1.7320508
        if dist == "DG":
            g = g * 2.23 + 21.33
        return g
    if dist == "T":
        return (_hash(seed, tag, rows, cols, 0) >> 28).to(torch.float32)
    if dist == "X":
        h = _hash(seed, tag, rows, cols, 0)
        u = _u24(_hash(seed, tag, rows, cols, 1))
        table = torch.tensor([0.0, -0.0, float("inf"), float("-inf"), float("nan"),
                              1e-45, -1e-45, 0.5], dtype=torch.float32, device=device)
        sel = (h & 15)
        special = table[torch.clamp(sel, max=7)]
        return torch.where(sel < 8, special, u)
    raise ValueError("unknown distribution %r" % dist)


def rows(dist: str, seed: int, row0: int, nrows: int, N: int, device="cpu",
         out: torch.Tensor | None = None) -> torch.Tensor:
    """Global rows [row0, row0+nrows) of an (infinitely tall) Q x N fp32 matrix."""
    if out is None:
        out = torch.empty((nrows, N), dtype=torch.float32, device=device)
    step = max(1, _CHUNK // max(N, 1))
    for a in range(0, nrows, step):
        b = min(nrows, a + step)
        r = torch.arange(row0 + a, row0 + b, device=out.device, dtype=torch.int64).unsqueeze(1)
        out[a:b] = _gen_block(dist, seed, r, N, out.device)
    return out


def row_subset(dist: str, seed: int, row_ids, N: int, device="cpu") -> torch.Tensor:
    """Arbitrary (sampled) global rows, bit-identical to those in rows()."""
    ids = torch.as_tensor(list(row_ids), dtype=torch.int64)
    out = torch.empty((len(ids), N), dtype=torch.float32, device=device)
    step = max(1, _CHUNK // max(N, 1))
    for a in range(0, len(ids), step):
        r = ids[a:a + step].to(device).unsqueeze(1)
        out[a:a + len(r)] = _gen_block(dist, seed, r, N, device)
    return out


def knn_points(kind: str, seed: int, row0: int, n: int, D: int, device="cpu") -> torch.Tensor:
    """n x D fp32 points: 'knn-U' uniform [0,1), 'knn-S' integers in [0,255]."""
    out = torch.empty((n, D), dtype=torch.float32, device=device)
    step = max(1, _CHUNK // max(D, 1))
    tag = _TAG[kind]
    cols = torch.arange(D, device=device, dtype=torch.int64).unsqueeze(0)
    for a in range(0, n, step):
        b = min(n, a + step)
        r = torch.arange(row0 + a, row0 + b, device=device, dtype=torch.int64).unsqueeze(1)
        h = _hash(seed, tag, r, cols, 0)
        if kind == "knn-U":
            out[a:b] = _u24(h)
        elif kind == "knn-S":
            # product of two bytes >> 8: integer in [0, 254], skewed towards 0
            out[a:b] = (((h & 255) * ((h >> 8) & 255)) >> 8).to(torch.float32)
        else:
            raise ValueError("unknown point kind %r" % kind)
    return out
