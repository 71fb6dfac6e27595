"""TEST INFRASTRUCTURE ONLY -- ctypes wrapper around the plain-C oracle (xro.c).

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with
the CUDA path; the op/dtype/mask codes below are re-declared on purpose and
cross-checked against the library header by tests/test_abi.py.

Parity status per function:
  reduce      pinned: P1-P11, P13, P16 (tests/test_oracle_pins.py)
  transform_reduce  pinned: P15 (lattice count by integer brute force, statistical pi),
              dot closed forms (tests/test_oracle_pins_n1.py)
  heat        pinned: P14 (hand-derived residuals in tests/golden/, invariants)
  (the paper prints no result value for any case: its Table 2 / Fig 11-12 are
  timings only, so paper *timings* are "parity unpinned" -- context only)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

OPS = {"+": 0, "*": 1, "max": 2, "min": 3, "&": 4, "|": 5, "^": 6, "&&": 7, "||": 8}
DTYPES = {"int32": 0, "int64": 1, "fp32": 2, "fp64": 3}
NP_DTYPES = {"int32": np.int32, "int64": np.int64, "fp32": np.float32, "fp64": np.float64}
GANG, WORKER, VECTOR, INIT_FROM_OUT = 0x1, 0x2, 0x4, 0x100
OK, ERR_INVALID, ERR_UNSUPPORTED = 0, 1, 2


class OracleError(RuntimeError):
    def __init__(self, status):
        super().__init__(f"oracle status {status}")
        self.status = status


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "xro.c")
    hdr = os.path.join(_HERE, "xro.h")
    newest = max(os.path.getmtime(src), os.path.getmtime(hdr))
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-ffp-contract=off", "-fno-fast-math",
                               "-shared", "-fPIC", src, "-o", _SO, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        i64p = ctypes.POINTER(ctypes.c_int64)
        vp = ctypes.c_void_p
        L.xro_out_count.argtypes = [i64p, ctypes.c_uint, i64p]
        L.xro_reduce.argtypes = [ctypes.c_int, ctypes.c_int, i64p, ctypes.c_uint, vp, vp, vp]
        L.xro_transform_reduce.argtypes = [ctypes.c_int, ctypes.c_int, i64p, ctypes.c_uint, vp, vp, vp, vp]
        L.xro_heat_init.argtypes = [ctypes.c_int64, ctypes.c_int64, vp]
        L.xro_heat.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, vp, vp, vp]
        _lib = L
    return _lib


def _dims(dims):
    return (ctypes.c_int64 * 3)(*[int(d) for d in dims])


def mask_of(levels) -> int:
    if isinstance(levels, int):
        return levels
    m = 0
    for ch in levels.lower():
        m |= {"g": GANG, "w": WORKER, "v": VECTOR}[ch]
    return m


def out_count(dims, levels) -> int:
    c = ctypes.c_int64(0)
    st = lib().xro_out_count(_dims(dims), mask_of(levels), ctypes.byref(c))
    if st:
        raise OracleError(st)
    return int(c.value)


def reduce_status(op, dtype, dims, mask) -> int:
    """Status code only (validation path), with dummy buffers."""
    cnt = 1
    out = np.zeros(max(cnt, 1), np.float64)
    return int(lib().xro_reduce(OPS[op] if isinstance(op, str) else op,
                                DTYPES[dtype] if isinstance(dtype, str) else dtype,
                                _dims(dims), mask, None, out.ctypes.data, None))


def reduce(op: str, dtype: str, dims, levels, x: np.ndarray, init: np.ndarray | None = None,
           want_abs: bool = False):
    """Oracle reduction of x (flattened nest dims) over ``levels``.

    Returns out (np array, dtype) or (out, abs_sum) when want_abs."""
    mask = mask_of(levels)
    dt = np.dtype(NP_DTYPES[dtype])
    x = np.ascontiguousarray(x, dtype=dt).reshape(-1)
    n = out_count(dims, mask)
    if init is not None:
        out = np.ascontiguousarray(np.asarray(init, dtype=dt).reshape(-1)).copy()
        assert out.size == n
        mask |= INIT_FROM_OUT
    else:
        out = np.zeros(n, dt)
    S = np.zeros(max(n, 1), np.float64)
    st = lib().xro_reduce(OPS[op], DTYPES[dtype], _dims(dims), mask,
                          x.ctypes.data if x.size else None,
                          out.ctypes.data if n else None, S.ctypes.data)
    if st:
        raise OracleError(st)
    return (out, S[:n]) if want_abs else out


XFORMS = {"disk": 1, "dot": 2}


def transform_reduce(xform: str, dtype: str, dims, levels, x: np.ndarray, y: np.ndarray,
                     init: np.ndarray | None = None, want_abs: bool = False):
    """N1 transform-reduce (see xro.h): 'disk' -> int64 counts, 'dot' -> dtype sums."""
    mask = mask_of(levels)
    dt = np.dtype(NP_DTYPES[dtype])
    x = np.ascontiguousarray(x, dtype=dt).reshape(-1)
    y = np.ascontiguousarray(y, dtype=dt).reshape(-1)
    n = out_count(dims, mask)
    odt = np.int64 if xform == "disk" else dt
    if init is not None:
        out = np.ascontiguousarray(np.asarray(init, dtype=odt).reshape(-1)).copy()
        mask |= INIT_FROM_OUT
    else:
        out = np.zeros(n, odt)
    S = np.zeros(max(n, 1), np.float64)
    st = lib().xro_transform_reduce(XFORMS[xform], DTYPES[dtype], _dims(dims), mask,
                                    x.ctypes.data if x.size else None, y.ctypes.data if y.size else None,
                                    out.ctypes.data if n else None, S.ctypes.data)
    if st:
        raise OracleError(st)
    return (out, S[:n]) if want_abs else out


def heat_init(nj: int, ni: int) -> np.ndarray:
    T = np.empty(nj * ni, np.float64)
    st = lib().xro_heat_init(nj, ni, T.ctypes.data)
    if st:
        raise OracleError(st)
    return T


def heat(nj: int, ni: int, iters: int, T: np.ndarray | None = None):
    """Run ``iters`` sweeps from T (default: heat_init).  Returns (T_final, residuals)."""
    T1 = heat_init(nj, ni) if T is None else np.array(T, np.float64).reshape(-1).copy()
    T2 = T1.copy()
    res = np.zeros(max(iters, 1), np.float64)
    st = lib().xro_heat(nj, ni, iters, T1.ctypes.data, T2.ctypes.data, res.ctypes.data)
    if st:
        raise OracleError(st)
    final = T1 if iters % 2 == 0 else T2
    return final, res[:iters]
