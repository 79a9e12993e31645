"""Seeded queue-bench item ids (an input generator; no queue arithmetic here).

The queue microbenchmark (BASELINE.json configs[1]) pushes
N unique 32-bit items through the queue. Item g (g = global item counter in
[0, N)) is `item_of(seed, g)`, a bijection on 32-bit integers, so every item
is unique by construction. The CUDA bench kernel computes the same function
on the device (`inputs/csrc/tqgen.cu` documents the twin); the oracle side
uses this one to form the expected multiset fingerprint.
"""
from __future__ import annotations

import numpy as np

from .graphs import _mix64

M32 = np.uint64(0xFFFFFFFF)


def seed32(seed: int) -> int:
    return int(_mix64(np.array([seed & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64))[0]) & 0xFFFFFFFF


def item_of(seed: int, g) -> np.ndarray:
    """Bijective 32-bit mix of the counter g (xor key, odd multiply, xorshift)."""
    x = (np.asarray(g, dtype=np.uint64) ^ np.uint64(seed32(seed))) & M32
    with np.errstate(over="ignore"):
        x = (x * np.uint64(0x9E3779B1)) & M32
        x ^= x >> np.uint64(16)
        x = (x * np.uint64(0x85EBCA6B)) & M32
        x ^= x >> np.uint64(13)
    return x.astype(np.uint32)


def fingerprint(items) -> tuple[int, int, int]:
    """(count, sum, xor) of splitmix64(item) over a multiset of items, mod 2**64."""
    items = np.asarray(items, dtype=np.uint64)
    f = _mix64(items)
    with np.errstate(over="ignore"):
        s = int(np.sum(f, dtype=np.uint64))
    x = int(np.bitwise_xor.reduce(f)) if f.size else 0
    return int(items.size), s, x
