"""Seeded synthetic inputs shared by tests/ and bench.py.

This module holds NO arithmetic of the method (no gcd, no index function, no
permutation): it only draws shapes and bit patterns, so that the oracle and the CUDA
path can be fed the same inputs without sharing code (DESIGN.md §"Input recipe").

Workload shapes follow PAPER.md and BASELINE.json:
  * config 1: m=1200, n=1800, 4-byte elements (BASELINE.json configs[0]);
  * config 2: the paper's GPU sweep, m, n uniform in [1000, 20000] (reading
    C14), 4- and 8-byte elements, seed 20140215;
  * config 3: skinny AoS of 2**26 structs x n in {2..32} 4-byte fields (BASELINE.json);
  * config 4: unit-stride AoS of 1..16-word structs (Fig. 8);
  * config 5: 4096 x 3000 fp32 batches and a ~140 GB fp64 matrix.
Element contents are random bit patterns (so float views contain NaN payloads, -0.0 and
subnormals): the transpose moves opaque words and must be bit exact.
"""
from __future__ import annotations

import numpy as np

SWEEP_SEED = 20140215
SWEEP_LO, SWEEP_HI = 1000, 20000

CONFIG1 = dict(m=1200, n=1800, elem_bytes=4)
CONFIG5B = dict(m=4096, n=3000, elem_bytes=4, batch=4096)
CONFIG5A = dict(m=120011, n=145820, elem_bytes=8)

_DTYPES = {1: np.uint8, 2: np.uint16, 4: np.uint32, 8: np.uint64}


def sweep_shapes(k: int, seed: int = SWEEP_SEED, lo: int = SWEEP_LO, hi: int = SWEEP_HI):
    """The first k shapes (m, n) of the config-2 sweep: uniform integers in [lo, hi]."""
    rng = np.random.default_rng(seed)
    mn = rng.integers(lo, hi + 1, size=(k, 2))
    return [(int(a), int(b)) for a, b in mn]


def random_words(count: int, elem_bytes: int, seed: int) -> np.ndarray:
    """`count` random elements of `elem_bytes` bytes as a numpy array.

    4/8-byte elements come back as uint32/uint64; 16-byte elements as a (count, 2)
    uint64 array (viewed flat as 2*count uint64); other multiples of 4 bytes (records)
    as a (count, elem_bytes // 4) uint32 array."""
    rng = np.random.default_rng(seed)
    if elem_bytes == 16:
        return rng.integers(0, 2**64, size=(count, 2), dtype=np.uint64, endpoint=False)
    if elem_bytes not in _DTYPES:  # records of elem_bytes / 4 random 32-bit words
        assert elem_bytes % 4 == 0
        return rng.integers(0, 2**32, size=(count, elem_bytes // 4), dtype=np.uint32, endpoint=False)
    dt = _DTYPES[elem_bytes]
    return rng.integers(0, np.iinfo(dt).max, size=count, dtype=dt, endpoint=True)


def fast_random_words(count: int, elem_bytes: int, seed: int) -> np.ndarray:
    """`count` random elements as a flat array of elem_bytes-byte words (uint32 / uint64, or
    uint8 for other sizes), drawn as raw bytes -- several times faster than random_words for
    the GB-sized full-comparison tests."""
    raw = np.frombuffer(np.random.default_rng(seed).bytes(count * elem_bytes), dtype=np.uint8)
    return raw.view({4: np.uint32, 8: np.uint64}.get(elem_bytes, np.uint8)).copy()


def index_words(count: int, elem_bytes: int) -> np.ndarray:
    """Element l holds the value l (readable diffs); 16-byte elements hold (l, ~l)."""
    if elem_bytes == 16:
        out = np.empty((count, 2), dtype=np.uint64)
        out[:, 0] = np.arange(count, dtype=np.uint64)
        out[:, 1] = ~out[:, 0]
        return out
    return np.arange(count, dtype=_DTYPES[elem_bytes])


def small_shapes(limit: int):
    """Every (m, n) with 1 <= m, n <= limit (brute-force coverage)."""
    return [(m, n) for m in range(1, limit + 1) for n in range(1, limit + 1)]


def skinny_field_counts():
    """config 3: n in {2, ..., 32}."""
    return list(range(2, 33))


def struct_words():
    """config 4: structs of 1..16 four-byte words."""
    return list(range(1, 17))
