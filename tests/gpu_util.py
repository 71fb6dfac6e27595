"""Helpers for the GPU parity tests: run the CUDA path through the C ABI and
compare with the oracle under the bars of SURVEY.md 8(c) / DESIGN.md:
  ints, & | ^, && ||, max/min : byte-equal (fp NaN == NaN, +-0 distinguished)
  fp '+'  : |gpu - ref| <= tau * S[o],  tau = 1e-5 (fp32) / 1e-12 (fp64), S = |init| + sum|x|
  fp '*'  : |gpu - ref| <= 1.01 * gamma_{n} * |ref| (+ one ulp of rounding the ref), n = segment + init
"""
from __future__ import annotations

import numpy as np

import oracle

TAU = {"fp32": 1e-5, "fp64": 1e-12}
UNIT = {"fp32": 2.0**-24, "fp64": 2.0**-53}
NP = oracle.NP_DTYPES
TORCH = None


def torch_dt(dtype):
    import torch
    return {"int32": torch.int32, "int64": torch.int64, "fp32": torch.float32,
            "fp64": torch.float64}[dtype]


def gpu_reduce(op, dtype, dims, levels, x: np.ndarray, init=None, offset: int = 0, stream=None):
    """Copy x to the device (optionally at an element offset inside a larger
    buffer, to exercise misaligned starts), reduce through the C ABI, return numpy."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    buf = torch.empty(x.size + offset + 1, dtype=torch_dt(dtype), device="cuda")
    dev = buf[offset:offset + x.size]
    dev.copy_(torch.from_numpy(np.ascontiguousarray(x)))
    n = xr.xr_out_count(dims, levels)
    out = torch.empty(max(n, 1), dtype=torch_dt(dtype), device="cuda")
    mask = xr.mask_of(levels)
    if init is not None:
        out[:n].copy_(torch.from_numpy(np.ascontiguousarray(init, dtype=NP[dtype])))
        mask |= xr.INIT_FROM_OUT
    s = torch.cuda.current_stream() if stream is None else stream
    st = xr.xr_reduce(op, dtype, dims, mask, dev.data_ptr() if x.size else 0, out.data_ptr(),
                      s.cuda_stream)
    if st != 0:
        raise xr.XReduceError(st, "xr_reduce")
    torch.cuda.synchronize()
    return out[:n].cpu().numpy()


def seg_len(dims, levels):
    m = oracle.mask_of(levels)
    L = 1
    for d in range(3):
        if (m >> d) & 1:
            L *= int(dims[d])
    return L


def check(op, dtype, dims, levels, gpu: np.ndarray, x: np.ndarray, init=None, exact=False):
    """Compare gpu with the oracle; returns the max |err| / bound ratio (0 if exact)."""
    ref, S = oracle.reduce(op, dtype, dims, levels, x, init=init, want_abs=True)
    assert gpu.shape == ref.shape, (gpu.shape, ref.shape)
    isfp = dtype.startswith("fp")
    if not isfp or op not in ("+", "*") or exact:
        if isfp:
            g, r = gpu.view(np.uint32 if dtype == "fp32" else np.uint64), \
                ref.view(np.uint32 if dtype == "fp32" else np.uint64)
            both_nan = np.isnan(gpu) & np.isnan(ref)
            bad = (g != r) & ~both_nan
        else:
            bad = gpu != ref
        if bad.any():
            i = int(np.flatnonzero(bad)[0])
            raise AssertionError(f"{op} {dtype} {dims} {levels}: mismatch at {i}: gpu={gpu[i]!r} "
                                 f"ref={ref[i]!r} ({int(bad.sum())} of {bad.size})")
        return 0.0
    g64, r64 = gpu.astype(np.float64), ref.astype(np.float64)
    fin = np.isfinite(r64)
    assert np.array_equal(np.isnan(g64), np.isnan(r64)), "NaN pattern differs"
    assert np.array_equal(g64[~fin & ~np.isnan(r64)], r64[~fin & ~np.isnan(r64)]), "inf differs"
    err = np.abs(g64[fin] - r64[fin])
    if op == "+":
        bound = TAU[dtype] * S[fin]
    else:
        n = seg_len(dims, levels) + (1 if init is not None else 0)
        u = UNIT[dtype]
        gam = n * u / (1 - n * u)
        bound = 1.01 * gam * np.abs(r64[fin]) + np.spacing(np.abs(r64[fin]).astype(NP[dtype])).astype(np.float64)
    ok = err <= bound
    if not ok.all():
        i = int(np.flatnonzero(~ok)[0])
        raise AssertionError(f"{op} {dtype} {dims} {levels}: |err| {err[i]:.3e} > bound {bound[i]:.3e} "
                             f"(gpu={g64[fin][i]!r}, ref={r64[fin][i]!r})")
    with np.errstate(divide="ignore", invalid="ignore"):
        ratio = np.where(bound > 0, err / bound, 0.0)
    return float(ratio.max()) if ratio.size else 0.0
