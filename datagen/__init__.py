"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no reduction, no combine):
it only maps (seed, global index) to input values via a counter-based
splitmix64 hash, implemented in ``gen.c`` (see its header for the formulas,
which follow SURVEY.md 8(d) "Generator").  Because values depend only on the
global index, a shard generated at ``start`` equals the slice of the full
array, which is what the multi-GPU tests rely on.

Workload recipes (value distributions per op, planted specials) live in
``datagen.recipes``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libxrgen.so")
_lib = None

BASE_SEED = 20140215  # PMAM'14 opening date


def build(force: bool = False) -> str:
    """Compile gen.c into libxrgen.so (plain gcc + OpenMP)."""
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=gnu11",
                               src, "-o", _SO])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u64, i64, vp = ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p
        L.xg_hash.restype = u64
        L.xg_hash.argtypes = [u64, u64]
        L.xg_splitmix64.restype = u64
        L.xg_splitmix64.argtypes = [u64]
        L.xg_hashes.argtypes = [u64, i64, i64, vp]
        L.xg_uniform_i32.argtypes = [u64, i64, i64, i64, i64, vp]
        L.xg_uniform_i64.argtypes = [u64, i64, i64, i64, i64, vp]
        L.xg_uniform_f32.argtypes = [u64, i64, i64, ctypes.c_double, ctypes.c_double, vp]
        L.xg_uniform_f64.argtypes = [u64, i64, i64, ctypes.c_double, ctypes.c_double, vp]
        L.xg_affine_i64.argtypes = [i64, i64, u64, u64, u64, vp]
        L.xg_affine_i32.argtypes = [i64, i64, u64, u64, u64, vp]
        L.xg_linear_i32.argtypes = [i64, i64, vp]
        L.xg_linear_i64.argtypes = [i64, i64, vp]
        L.xg_select.argtypes = [u64, i64, i64, u64, u64, vp]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def splitmix64(x: int) -> int:
    return int(lib().xg_splitmix64(ctypes.c_uint64(x & (2**64 - 1))))


def case_seed(cfg: int, op: int, dtype: int, mask: int, variant: int = 0) -> int:
    """Per-case seed: splitmix64(BASE ^ cfg<<40 ^ op<<32 ^ dtype<<24 ^ mask<<16 ^ variant)."""
    x = BASE_SEED ^ (cfg << 40) ^ (op << 32) ^ (dtype << 24) ^ (mask << 16) ^ variant
    return splitmix64(x)


def hashes(seed: int, n: int, start: int = 0) -> np.ndarray:
    out = np.empty(n, np.uint64)
    lib().xg_hashes(seed, start, n, _p(out))
    return out


def uniform_int(seed: int, n: int, lo: int, hi: int, dtype, start: int = 0) -> np.ndarray:
    dt = np.dtype(dtype)
    out = np.empty(n, dt)
    if dt == np.int32:
        lib().xg_uniform_i32(seed, start, n, lo, hi, _p(out))
    elif dt == np.int64:
        lib().xg_uniform_i64(seed, start, n, lo, hi, _p(out))
    else:
        raise TypeError(dt)
    return out


def uniform_float(seed: int, n: int, lo: float, hi: float, dtype, start: int = 0) -> np.ndarray:
    dt = np.dtype(dtype)
    out = np.empty(n, dt)
    if dt == np.float32:
        lib().xg_uniform_f32(seed, start, n, lo, hi, _p(out))
    elif dt == np.float64:
        lib().xg_uniform_f64(seed, start, n, lo, hi, _p(out))
    else:
        raise TypeError(dt)
    return out


def linear(n: int, dtype, start: int = 0) -> np.ndarray:
    """Global linear index (start + t), wrapped to the dtype width for ints."""
    dt = np.dtype(dtype)
    if dt == np.int32:
        out = np.empty(n, dt)
        lib().xg_linear_i32(start, n, _p(out))
        return out
    if dt == np.int64:
        out = np.empty(n, dt)
        lib().xg_linear_i64(start, n, _p(out))
        return out
    return (np.arange(start, start + n, dtype=np.float64)).astype(dt)


def affine_perm(n_total: int, n: int, dtype, a: int, b: int, start: int = 0) -> np.ndarray:
    """(a*idx + b) mod n_total for idx in [start, start+n): a permutation of
    0..n_total-1 when gcd(a, n_total) = 1."""
    dt = np.dtype(dtype)
    out = np.empty(n, dt)
    if dt == np.int64:
        lib().xg_affine_i64(start, n, a, b, n_total, _p(out))
    elif dt == np.int32:
        lib().xg_affine_i32(start, n, a, b, n_total, _p(out))
    else:
        tmp = np.empty(n, np.int64)
        lib().xg_affine_i64(start, n, a, b, n_total, _p(tmp))
        out = tmp.astype(dt)
    return out


def select(seed: int, n: int, num: int, den: int, start: int = 0) -> np.ndarray:
    """Bernoulli(num/den) boolean mask at global indices [start, start+n)."""
    out = np.empty(n, np.uint8)
    lib().xg_select(seed, start, n, num, den, _p(out))
    return out.view(np.bool_)
