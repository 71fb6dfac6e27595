"""All-cores OpenMP CPU baseline, a ctypes wrapper of omp.c.

A timed BASELINE for bench.py, beside the single-thread oracle: it is neither
the oracle (oracle/) nor the product (the CUDA path), shares no code with
either, and is checked against the oracle by tests/test_cpubase.py.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libxrbase.so")
_lib = None

OPS = {"+": 0, "*": 1, "max": 2, "min": 3, "&": 4, "|": 5, "^": 6, "&&": 7, "||": 8}
DTYPES = {"int32": 0, "int64": 1, "fp32": 2, "fp64": 3}
NP = {"int32": np.int32, "int64": np.int64, "fp32": np.float32, "fp64": np.float64}


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "omp.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-ffp-contract=off",
                               "-std=gnu11", "-shared", "-fPIC", src, "-o", _SO, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        L.xrb_reduce.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_int64),
                                 ctypes.c_uint, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
        L.xrb_num_procs.restype = ctypes.c_int
        _lib = L
    return _lib


def num_procs() -> int:
    return int(lib().xrb_num_procs())


def mask_of(levels: str) -> int:
    return sum({"g": 1, "w": 2, "v": 4}[c] for c in levels.lower())


def reduce(op: str, dtype: str, dims, levels: str, x: np.ndarray, init=None, threads: int = 0):
    dims = [int(d) for d in dims]
    kept = [d for b, d in zip((1, 2, 4), dims) if not mask_of(levels) & b]
    cnt = int(np.prod(kept)) if kept else 1
    mask = mask_of(levels)
    if init is not None:
        out = np.ascontiguousarray(np.asarray(init, NP[dtype]).reshape(-1)).copy()
        mask |= 0x100
    else:
        out = np.zeros(cnt, NP[dtype])
    x = np.ascontiguousarray(x, NP[dtype]).reshape(-1)
    st = lib().xrb_reduce(OPS[op], DTYPES[dtype], (ctypes.c_int64 * 3)(*dims), mask,
                          x.ctypes.data, out.ctypes.data, int(threads))
    if st:
        raise RuntimeError(f"cpubase status {st}")
    return out
