"""Workload recipes: value distributions per op, shaped like the paper's workloads.

Holds no reduction arithmetic.  Every recipe maps global indices
[start, start+n) of a nest to values, so shards are exact slices.  The
recipes follow SURVEY.md 8(d) (cfg1..cfg5 table): planted values are placed at
hash-chosen indices at a rate scaled to the segment length L (the product of
the reduced extents) so that every segment stays non-trivial.

Recipe names (``kind``):
  ints      U_int[-1000,1000] (ints) / U[-1,1) (floats)
  linear    global linear index (P1 closed form)
  ones      all ones (P2)
  u01       U[0,1)   (worst relative case for fp sums)
  um11      U[-1,1)
  intvals   integer-valued {-16..16}; fp sums are exact in any order (P8)
  maxmin    U[-1,1) with planted +2 / -2 at rate ~1/L (floats); an affine
            permutation of 0..N-1 (ints) (P4)
  mul       ints: +-1 with +-3 at rate 1/64 (P5); floats: random sign x 1 with
            planted 2.0 and 0.5 at rate ~50/L each -> exact power of two (P9)
  mulgen    U[0.999, 1.001] (general fp products, C10 bound)
  band      ~0 with ~4 planted ~(1<<r) per segment (P6)
  bor       0 with ~4 planted 1<<r per segment (P6)
  bxor      uniform bits (P3 via ``linear``)
  land      non-zero with zeros (incl. -0.0) at rate 0.7/L (P7)
  lor       zeros (+-0.0) with non-zeros at rate 0.7/L (P7)
  specials  U[-1,1) with NaN, +-inf, +-0, subnormals planted (floats only)
  mulspecials  the ``mul`` recipe (exact power-of-two products) with NaN, +-inf,
            +-0 planted -- products of specials without intermediate
            under/overflow, the only regime where products are order independent
"""
from __future__ import annotations

import numpy as np

from . import affine_perm, linear, select, splitmix64, uniform_float, uniform_int, hashes

_DT = {"int32": np.int32, "int64": np.int64, "fp32": np.float32, "fp64": np.float64}
_RATE_DEN = 1 << 24


def np_dtype(dtype) -> np.dtype:
    if isinstance(dtype, str):
        return np.dtype(_DT[dtype])
    return np.dtype(dtype)


def seg_len(dims, mask) -> int:
    L = 1
    for d in range(3):
        if (mask >> d) & 1:
            L *= int(dims[d])
    return max(L, 1)


def _sub(seed: int, k: int) -> int:
    return splitmix64(seed ^ (0xA5A5_0000 + k))


def _rate(seed, n, start, per_seg: float, L: int) -> np.ndarray:
    num = int(min(_RATE_DEN, max(1, round(per_seg * _RATE_DEN / L))))
    return select(seed, n, num, _RATE_DEN, start)


def make(kind: str, dims, mask: int, dtype, seed: int, start: int = 0, n: int | None = None) -> np.ndarray:
    """Flattened input values at global indices [start, start+n) of nest ``dims``."""
    dt = np_dtype(dtype)
    N = int(dims[0]) * int(dims[1]) * int(dims[2])
    if n is None:
        n = N - start
    L = seg_len(dims, mask)
    isint = dt.kind == "i"
    bits = dt.itemsize * 8

    if kind == "ints":
        return uniform_int(seed, n, -1000, 1000, dt, start) if isint else \
            uniform_float(seed, n, -1.0, 1.0, dt, start)
    if kind == "linear":
        return linear(n, dt, start)
    if kind == "ones":
        return np.ones(n, dt)
    if kind == "u01":
        return uniform_float(seed, n, 0.0, 1.0, dt, start)
    if kind == "um11":
        return uniform_float(seed, n, -1.0, 1.0, dt, start)
    if kind == "intvals":
        v = uniform_int(seed, n, -16, 16, np.int64, start)
        return v.astype(dt)
    if kind == "maxmin":
        if isint:
            # affine bijection of 0..N-1 with an odd multiplier coprime to N
            a = 0x9E3779B1 | 1
            while np.gcd(a, N) != 1:
                a += 2
            return affine_perm(N, n, dt, a % N if N > 1 else 1, 12345 % max(N, 1), start)
        x = uniform_float(seed, n, -1.0, 1.0, dt, start)
        x[_rate(_sub(seed, 1), n, start, 1.0, L)] = 2.0
        x[_rate(_sub(seed, 2), n, start, 1.0, L)] = -2.0
        return x
    if kind == "mul":
        if isint:
            sgn = uniform_int(_sub(seed, 3), n, 0, 1, np.int64, start) * 2 - 1
            three = _rate(_sub(seed, 4), n, start, L / 64.0, L)
            return (sgn * np.where(three, 3, 1)).astype(dt)
        sgn = uniform_int(_sub(seed, 3), n, 0, 1, np.int64, start) * 2 - 1
        x = sgn.astype(dt)
        per = min(50.0, L / 8.0)
        two = _rate(_sub(seed, 5), n, start, per, L)
        half = _rate(_sub(seed, 6), n, start, per, L) & ~two
        x[two] *= 2.0
        x[half] *= 0.5
        return x
    if kind == "mulgen":
        return uniform_float(seed, n, 0.999, 1.001, dt, start)
    if kind in ("band", "bor"):
        r = (hashes(_sub(seed, 7), n, start) % np.uint64(bits)).astype(np.int64)
        one_hot = np.left_shift(np.ones(n, np.uint64), r.astype(np.uint64))
        plant = _rate(_sub(seed, 8), n, start, 4.0, L)
        if kind == "bor":
            u = np.where(plant, one_hot, np.uint64(0))
        else:
            u = np.where(plant, ~one_hot, np.uint64(2**64 - 1))
        if bits == 32:
            return (u & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)
        return u.view(np.int64)
    if kind == "bxor":
        h = hashes(seed, n, start)
        if bits == 32:
            return (h >> np.uint64(32)).astype(np.uint32).view(np.int32)
        return h.view(np.int64)
    if kind in ("land", "lor"):
        special = _rate(_sub(seed, 9), n, start, 0.7, L)
        negz = (hashes(_sub(seed, 10), n, start) & np.uint64(1)).astype(bool)
        if isint:
            nz = uniform_int(seed, n, 1, 1000, dt, start)
            zero = np.zeros(n, dt)
        else:
            nz = uniform_float(seed, n, 0.5, 1.5, dt, start)
            zero = np.where(negz, dt.type(-0.0), dt.type(0.0)).astype(dt)
        if kind == "land":
            return np.where(special, zero, nz).astype(dt)
        return np.where(special, nz, zero).astype(dt)
    if kind == "specials":
        if isint:
            raise ValueError("specials is a floating-point recipe")
        x = uniform_float(seed, n, -1.0, 1.0, dt, start)
        h = hashes(_sub(seed, 11), n, start)
        pick = (h % np.uint64(16)).astype(np.int64)
        tiny = np.finfo(dt).smallest_subnormal
        table = [np.nan, np.inf, -np.inf, 0.0, -0.0, tiny, -tiny]
        plant = _rate(_sub(seed, 12), n, start, 3.0, L)
        for k, v in enumerate(table):
            x[plant & (pick == k)] = v
        return x
    if kind == "mulspecials":
        if isint:
            raise ValueError("mulspecials is a floating-point recipe")
        x = make("mul", dims, mask, dtype, seed, start, n)
        h = hashes(_sub(seed, 13), n, start)
        pick = (h % np.uint64(8)).astype(np.int64)
        plant = _rate(_sub(seed, 14), n, start, 2.0, L)
        for k, v in enumerate([np.nan, np.inf, -np.inf, 0.0, -0.0]):
            x[plant & (pick == k)] = v
        return x
    raise ValueError(f"unknown recipe {kind!r}")
