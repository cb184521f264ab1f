"""Seeded synthetic inputs shared by the tests, smoke() and bench.py.

This is the ONLY module both the CUDA path's callers and the oracle consume.  It holds no
Paillier, Montgomery, Philox or codec arithmetic — only seeded draws with the shapes and value
distributions of the paper's workloads (DESIGN.md §4 "input recipe"), plus limb-array
marshalling (little-endian 32-bit words, the ABI layout).

Workload shapes (BASELINE.json ``configs``; PAPER L375 models, L432 settings, Table II):
  C1  1024-bit key, 1,000 fixed-point values a, b ~ U(-0.5, 0.5)
  C2  Homo LR: 8 clients x 1,048,576-element gradients ~ N(0, 0.05^2), clipped to +-1,
      1 % of entries exactly +-1 (Avazu has 1,000,000 features, L314)
  C3  Hetero LR: 4,194,304 residuals ~ U(-1, 1) and F = 8 per-feature u32 scalars
  C4  Hetero SBT: 1,048,576 samples, (g, h) = (p - y, p(1 - p)), 256 quantile bins
  C5  key sweep: plaintexts uniform in [0, n)
"""

from __future__ import annotations

import random
from typing import List, Sequence, Tuple

import numpy as np


# ----------------------------------------------------------------------------- limb marshalling


def ints_to_limbs(values: Sequence[int], words: int) -> np.ndarray:
    """Python ints -> uint32 array [len(values), words], little-endian limbs."""
    out = np.zeros((len(values), words), dtype=np.uint32)
    for i, v in enumerate(values):
        v = int(v)
        if v < 0 or v >> (32 * words):
            raise ValueError("value does not fit in %d limbs" % words)
        b = v.to_bytes(4 * words, "little")
        out[i] = np.frombuffer(b, dtype="<u4")
    return out


def limbs_to_ints(arr: np.ndarray) -> List[int]:
    """uint32/int32 array [count, words] -> Python ints."""
    a = np.ascontiguousarray(arr).view(np.uint32)
    return [int.from_bytes(row.astype("<u4").tobytes(), "little") for row in a]


# ----------------------------------------------------------------------------- big-integer draws


def uniform_below(bound: int, count: int, seed: int) -> List[int]:
    """``count`` integers uniform in [0, bound) (C5: m ~ U[0, n))."""
    rng = random.Random(seed)
    return [rng.randrange(bound) for _ in range(count)]


def uniform_words(count: int, words: int, seed: int) -> np.ndarray:
    """Uniform random uint32 limbs [count, words]."""
    g = np.random.default_rng(seed)
    return g.integers(0, 1 << 32, size=(count, words), dtype=np.uint64).astype(np.uint32)


# ----------------------------------------------------------------------------- float workloads


def c1_values(n: int = 1000) -> Tuple[np.ndarray, np.ndarray]:
    """C1: a, b ~ U(-0.5, 0.5) float32 (seeds 1 and 2)."""
    a = np.random.default_rng(1).uniform(-0.5, 0.5, n).astype(np.float32)
    b = np.random.default_rng(2).uniform(-0.5, 0.5, n).astype(np.float32)
    return a, b


def c2_gradient(client: int, n: int = 1 << 20) -> np.ndarray:
    """C2: one client's gradient ~ N(0, 0.05^2), clipped to +-1, 1 % of entries exactly +-1."""
    g = np.random.default_rng(20 + client)
    x = np.clip(g.normal(0.0, 0.05, n), -1.0, 1.0)
    k = n // 100
    pos = g.choice(n, size=k, replace=False)
    x[pos] = np.where(g.random(k) < 0.5, -1.0, 1.0)
    return x.astype(np.float32)


def c3_residuals(n: int = 1 << 22, features: int = 8, seed: int = 30) -> Tuple[np.ndarray, np.ndarray]:
    """C3: residuals d ~ U(-1, 1) float32 [n] and per-feature unsigned scalars [n, F] (u32)."""
    g = np.random.default_rng(seed)
    d = g.uniform(-1.0, 1.0, n).astype(np.float32)
    x = g.integers(0, 1 << 32, size=(n, features), dtype=np.uint64).astype(np.uint32)
    return d, x


def c4_histogram(n: int = 1 << 20, bins: int = 256, skew: bool = False,
                 seed: int = 40) -> Tuple[np.ndarray, np.ndarray, np.ndarray, np.ndarray]:
    """C4: interleaved (g, h) float32 [2n], per-sample bin ids, CSR offsets [bins+1], idx [n].

    y ~ Bernoulli(0.5), p ~ U(0, 1), g = p - y, h = p(1 - p).  Bins are the 256 quantile bins of
    a N(0, 1) feature; ``skew`` draws Zipf(1.2)-distributed bins instead.
    """
    r = np.random.default_rng(seed)
    y = (r.random(n) < 0.5).astype(np.float64)
    p = r.random(n)
    gh = np.empty(2 * n, dtype=np.float32)
    gh[0::2] = (p - y).astype(np.float32)
    gh[1::2] = (p * (1.0 - p)).astype(np.float32)
    if skew:
        b = (r.zipf(1.2, n) - 1) % bins
    else:
        f = r.normal(0.0, 1.0, n)
        edges = np.quantile(f, np.linspace(0, 1, bins + 1)[1:-1])
        b = np.searchsorted(edges, f, side="right")
    b = b.astype(np.int64)
    idx = np.argsort(b, kind="stable").astype(np.int64)
    counts = np.bincount(b, minlength=bins)
    offsets = np.zeros(bins + 1, dtype=np.int64)
    offsets[1:] = np.cumsum(counts)
    return gh, b, offsets, idx


def random_segments(total: int, segments: int, seed: int, empty_frac: float = 0.1) -> np.ndarray:
    """Ragged CSR offsets [segments+1] over ``total`` items with some empty segments."""
    r = np.random.default_rng(seed)
    cuts = np.sort(r.integers(0, total + 1, size=segments - 1))
    offs = np.concatenate([[0], cuts, [total]]).astype(np.int64)
    # force a few empty segments by duplicating cut points
    k = int(segments * empty_frac)
    if k and segments > 2:
        for j in r.choice(np.arange(1, segments), size=min(k, segments - 1), replace=False):
            offs[j] = offs[j - 1]
        offs = np.maximum.accumulate(offs)
    return offs
