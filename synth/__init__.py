"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no stencil, no model): it only
turns (seed, global index) into an fp32 value, so that the CPU oracle and the
CUDA path are fed bit-identical fields and every rank of a slab decomposition
can regenerate its own rows from global indices.

Recipe:
    key   = global_linear_index XOR (seed * 0xD1B54A32D192ED03)   (mod 2**64)
    z     = splitmix64(key)
    value = (z >> 40) * 2**-24            -> fp32 in [0, 1), exactly representable

The paper's workloads are dense random fields on cubes/squares (PAPER.md
L1179-1195, §5); the ring (the fixed boundary, reading R2) is part of
the field and uses the same generator.
"""
from __future__ import annotations

import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_SEED_MIX = 0xD1B54A32D192ED03

# Per-config seeds: C1..C5 -> 1..5
CONFIG_SEEDS = {"C1": 1, "C2": 2, "C3": 3, "C4": 4, "C5": 5, "X1": 7, "W1": 8, "X2": 9}


def _splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def uniform_flat(seed: int, start: int, count: int, out: np.ndarray | None = None,
                 chunk: int = 1 << 24) -> np.ndarray:
    """fp32 values for global linear indices [start, start+count)."""
    if out is None:
        out = np.empty(count, dtype=np.float32)
    key = np.uint64((seed * _SEED_MIX) & 0xFFFFFFFFFFFFFFFF)
    scale = np.float32(2.0 ** -24)
    for off in range(0, count, chunk):
        n = min(chunk, count - off)
        idx = np.arange(start + off, start + off + n, dtype=np.uint64)
        z = _splitmix64(idx ^ key)
        out[off:off + n] = (z >> np.uint64(40)).astype(np.float32) * scale
    return out


def field(seed: int, dims, row_start: int = 0, nrows: int | None = None) -> np.ndarray:
    """Random field of full extents `dims` (S1 outermost, row-major), or the
    slab of rows [row_start, row_start+nrows) along S1, generated from global
    indices so any slab equals the corresponding rows of the whole field."""
    dims = tuple(int(d) for d in dims)
    if nrows is None:
        nrows = dims[0] - row_start
    plane = int(np.prod(dims[1:], dtype=np.int64))
    flat = uniform_flat(seed, row_start * plane, nrows * plane)
    return flat.reshape((nrows,) + dims[1:])


def pinned_field(seed: int, dims):
    """Same field in pinned host memory (torch), for the e2e bench leg."""
    import torch
    a = field(seed, dims)
    t = torch.empty(a.shape, dtype=torch.float32, pin_memory=True)
    t.numpy()[...] = a
    return t
