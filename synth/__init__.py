"""Seeded synthetic inputs shared by the oracle-side tests and the CUDA-side tests.

This module is deliberately *outside* both ``oracle/`` and the product package:
it holds only a counter-based random generator (splitmix64) and the workload
recipes of DESIGN.md §"Input recipe" — none of the method's arithmetic (no
reduction, no schedule, no stencil).  Both sides receive the same host arrays.

Every value is ``f(seed, rank, epoch, index)`` so that any element of a full-size
input can be regenerated on its own (sampled parity at BASELINE sizes).
"""
from __future__ import annotations

import numpy as np

BASE_SEED = 0x5C24  # SURVEY §8(d) "Seeds: base 0x5C24"

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def _mix(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        return z ^ (z >> np.uint64(31))


def _key(seed: int, rank: int, epoch: int) -> np.uint64:
    with np.errstate(over="ignore"):
        k = _mix(np.array([seed & 0xFFFFFFFFFFFFFFFF], dtype=np.uint64))
        k = _mix(k ^ (np.uint64(rank + 1) * _GOLDEN))
        k = _mix(k ^ (np.uint64(epoch + 1) * _C1))
    return k[0]


def u64(seed: int, rank: int, epoch: int, n: int, start: int = 0) -> np.ndarray:
    """n raw 64-bit values for indices [start, start+n)."""
    idx = np.arange(start, start + n, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _mix(_key(seed, rank, epoch) + (idx + np.uint64(1)) * _GOLDEN)


def u64_at(seed: int, rank: int, epoch: int, idx: np.ndarray) -> np.ndarray:
    """Raw values at arbitrary indices (for sampled checks at full size)."""
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _mix(_key(seed, rank, epoch) + (idx + np.uint64(1)) * _GOLDEN)


def _unit(raw: np.ndarray) -> np.ndarray:
    """float64 in [0, 1) from the top 53 bits."""
    return (raw >> np.uint64(11)).astype(np.float64) * (1.0 / (1 << 53))


def uniform_f32(seed, rank, epoch, n, lo=-1.0, hi=1.0, start=0) -> np.ndarray:
    return (lo + (hi - lo) * _unit(u64(seed, rank, epoch, n, start))).astype(np.float32)


def normal_f32(seed, rank, epoch, n, sigma=1.0, start=0) -> np.ndarray:
    """Box-Muller N(0, sigma^2) in fp32 (DL-gradient-like values)."""
    raw = u64(seed, rank, epoch, 2 * n, 2 * start)
    u1 = _unit(raw[0::2])
    u2 = _unit(raw[1::2])
    r = np.sqrt(-2.0 * np.log1p(-u1))
    return (sigma * r * np.cos(2.0 * np.pi * u2)).astype(np.float32)


def normal_f32_at(seed, rank, epoch, idx, sigma=1.0) -> np.ndarray:
    idx = np.asarray(idx, dtype=np.uint64)
    u1 = _unit(u64_at(seed, rank, epoch, 2 * idx))
    u2 = _unit(u64_at(seed, rank, epoch, 2 * idx + np.uint64(1)))
    r = np.sqrt(-2.0 * np.log1p(-u1))
    return (sigma * r * np.cos(2.0 * np.pi * u2)).astype(np.float32)


def int32_range(seed, rank, epoch, n, lo, hi, start=0) -> np.ndarray:
    """Uniform int32 in [lo, hi)."""
    span = np.uint64(hi - lo)
    return ((u64(seed, rank, epoch, n, start) % span).astype(np.int64) + lo).astype(np.int32)


def int32_full(seed, rank, epoch, n, start=0) -> np.ndarray:
    """All 2^32 bit patterns equally likely (exercises wrap-around)."""
    return (u64(seed, rank, epoch, n, start) >> np.uint64(32)).astype(np.uint32).view(np.int32)


def int_valued_f32(seed, rank, epoch, n, bound, start=0) -> np.ndarray:
    """Integer-valued fp32 with |x| < bound: every summation order is exact when
    P*bound <= 2^24 (SURVEY §8(c).3 pin "fp32 allreduce with integer-valued inputs")."""
    return int32_range(seed, rank, epoch, n, -bound + 1, bound, start).astype(np.float32)


def bytes_tagged(seed, rank, epoch, nbytes) -> np.ndarray:
    """Epoch-tagged payload bytes: value(e, r, i) = splitmix64(seed, r, e, i)
    (SURVEY §8(c).3 "No early or stale visibility")."""
    n64 = (nbytes + 7) // 8
    return u64(seed, rank, epoch, n64).view(np.uint8)[:nbytes].copy()


def permutation(seed, rank, epoch, n) -> np.ndarray:
    """Seeded permutation of range(n) (Pready orders, block->partition maps)."""
    return np.argsort(u64(seed, rank, epoch, n), kind="stable").astype(np.int32)


# ---------------------------------------------------------------------------
# Workload shapes: DL-gradient tensor sizes.
# ---------------------------------------------------------------------------
RESNET50_SIZES = (
    [64] * 14 + [128] * 16 + [256] * 32 + [512] * 22 + [1000] + [1024] * 14 + [2048] * 8
    + [4096] + [9408] + [16384] * 6 + [32768] + [36864] * 3 + [65536] * 7 + [131072] * 2
    + [147456] * 4 + [262144] * 11 + [524288] * 2 + [589824] * 6 + [1048576] * 5 + [2048000]
    + [2097152] + [2359296] * 3
)
BERT_LARGE_SIZES = (
    [1024] * 219 + [2048] + [4096] * 24 + [524288] + [1048576] * 97 + [4194304] * 48 + [31254528]
)


def jacobi_init(ny: int, nx: int, kind: str = "perf", seed: int = BASE_SEED) -> np.ndarray:
    """Initial fp32 grid (boundary included).  'perf': interior 0, top row 1.0,
    other edges 0.  'random': uniform [0,1) everywhere."""
    if kind == "perf":
        a = np.zeros((ny, nx), dtype=np.float32)
        a[0, :] = 1.0
        return a
    if kind == "random":
        return uniform_f32(seed, 0, 0, ny * nx, 0.0, 1.0).reshape(ny, nx)
    raise ValueError(kind)


def uniform_f32_at(seed, rank, epoch, idx, lo=-1.0, hi=1.0) -> np.ndarray:
    """uniform_f32 values at arbitrary indices (sampled parity at full size)."""
    return (lo + (hi - lo) * _unit(u64_at(seed, rank, epoch, idx))).astype(np.float32)


def normal_f64(seed, rank, epoch, n, sigma=1.0, start=0) -> np.ndarray:
    """Box-Muller N(0, sigma^2) kept in float64 (fp64 allreduce inputs)."""
    raw = u64(seed, rank, epoch, 2 * n, 2 * start)
    u1 = _unit(raw[0::2])
    u2 = _unit(raw[1::2])
    return sigma * np.sqrt(-2.0 * np.log1p(-u1)) * np.cos(2.0 * np.pi * u2)


def bf16_bits(seed, rank, epoch, n, sigma=1.0, start=0) -> np.ndarray:
    """bf16 inputs as uint16 bit patterns: the upper half of normal_f32's bits
    (truncation is part of the random draw, not of the method)."""
    return (normal_f32(seed, rank, epoch, n, sigma, start).view(np.uint32) >> np.uint32(16)).astype(np.uint16)


def bf16_bits_raw(seed, rank, epoch, n, start=0) -> np.ndarray:
    """Arbitrary finite bf16 bit patterns (every exponent incl. subnormals)."""
    b = (u64(seed, rank, epoch, n, start) >> np.uint64(48)).astype(np.uint16)
    exp = (b >> np.uint16(7)) & np.uint16(0xFF)
    return np.where(exp == 0xFF, b & np.uint16(0xBFFF), b).astype(np.uint16)  # no inf/NaN


def bce_inputs(seed, rank, epoch, n, start=0):
    """DL proxy inputs (R28): predictions p uniform in [0.02, 0.98) (post-sigmoid
    probabilities away from 0/1) and binary targets y in {0, 1}."""
    raw = u64(seed, rank, epoch, 2 * n, 2 * start)
    p = (0.02 + 0.96 * _unit(raw[0::2])).astype(np.float32)
    y = (raw[1::2] >> np.uint64(63)).astype(np.float32)
    return p, y
