#!/usr/bin/env python3
"""Kernel driver for profiling and per-shape timing (not a bench line).

  python tools/kdriver.py CASE [--reps R] [--time]

CASE names a BASELINE config shape, e.g. cfg2-f32-sum, cfg2-i64-sum, cfg3-row,
cfg3-col, cfg4-heat, cfg5-<op>-<dtype>-<mask>, cfg1-<mask>, or any nest
nest-<op>-<dtype>-<n0>x<n1>x<n2>-<mask>.  --cold flushes L2 (a 256 MiB write)
before every timed call (cfg1 "cold" latency).  Inputs are random
device tensors (values do not change the memory traffic).  With --time, prints
a JSON line per case with the CUDA-event kernel time, algorithmic bytes and
GB/s vs the measured HBM peak.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

TDT = {"int32": torch.int32, "int64": torch.int64, "fp32": torch.float32, "fp64": torch.float64}
SIZE = {"int32": 4, "int64": 8, "fp32": 4, "fp64": 8}


def tensor(n, dtype):
    if dtype.startswith("fp"):
        return torch.rand(n, dtype=TDT[dtype], device="cuda")
    return torch.randint(-1000, 1000, (n,), dtype=TDT[dtype], device="cuda")


def cases(name):
    """-> list of (label, op, dtype, dims, levels)"""
    if name.startswith("cfg2-"):
        _, dt, op = name.split("-")
        dtype = {"f32": "fp32", "i64": "int64", "f64": "fp64", "i32": "int32"}[dt]
        return [(name, {"sum": "+", "max": "max", "min": "min", "prod": "*"}[op], dtype, (1 << 30, 1, 1), "gwv")]
    if name == "cfg3-row":
        return [(name, "+", "fp32", (32768, 1, 32768), "v")]
    if name == "cfg3-col":
        return [(name, "+", "fp32", (1, 32768, 32768), "w")]
    if name.startswith("cfg1-"):
        return [(name, "+", "int32", (64, 64, 128), name.split("-")[1])]
    if name == "cfg5-all":
        out = []
        for dtype in ["int32", "int64", "fp32", "fp64"]:
            for op in ["*", "&", "|", "^", "&&", "||"]:
                if dtype.startswith("fp") and op in "&|^":
                    continue
                for lv in ["g", "w", "v", "gw", "gv", "wv", "gwv"]:
                    out.append((f"cfg5-{op}-{dtype}-{lv}", op, dtype, (512, 512, 512), lv))
        return out
    if name.startswith("cfg5-"):
        _, op, dtype, lv = name.split("-")
        op = {"mul": "*", "and": "&", "or": "|", "xor": "^", "land": "&&", "lor": "||", "add": "+",
              "max": "max", "min": "min"}[op]
        return [(name, op, dtype, (512, 512, 512), lv)]
    if name.startswith("nest-"):  # nest-<op>-<dtype>-<n0>x<n1>x<n2>-<mask>, op as in cfg5
        _, op, dtype, dims, lv = name.split("-")
        op = {"mul": "*", "and": "&", "or": "|", "xor": "^", "land": "&&", "lor": "||", "add": "+",
              "max": "max", "min": "min"}[op]
        return [(name, op, dtype, tuple(int(d) for d in dims.split("x")), lv)]
    raise SystemExit(f"unknown case {name}")


def peak():
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        return 6650.0


_FLUSH = None


def flush_l2():
    global _FLUSH
    if _FLUSH is None:
        _FLUSH = torch.empty(64 << 20, dtype=torch.float32, device="cuda")  # 256 MiB > 126 MB L2
    _FLUSH.fill_(1.0)


def run_reduce(label, op, dtype, dims, lv, reps, timed, cache, cold=False):
    n = dims[0] * dims[1] * dims[2]
    key = (dtype, n)
    if key not in cache:
        cache.clear()
        torch.cuda.empty_cache()
        cache[key] = tensor(n, dtype)
    x = cache[key]
    cnt = xr.xr_out_count(dims, lv)
    out = torch.zeros(cnt, dtype=TDT[dtype], device="cuda")
    s = torch.cuda.current_stream()
    for _ in range(3):
        assert xr.xr_reduce(op, dtype, dims, lv, x.data_ptr(), out.data_ptr(), s.cuda_stream) == 0
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        if cold:
            flush_l2()
        a.record(s)
        xr.xr_reduce(op, dtype, dims, lv, x.data_ptr(), out.data_ptr(), s.cuda_stream)
        b.record(s)
    torch.cuda.synchronize()
    if timed:
        ms = sorted(a.elapsed_time(b) for a, b in evs)
        med = ms[len(ms) // 2]
        byts = (n + cnt) * SIZE[dtype]
        plan = xr.xr_plan_describe(op, dtype, dims, lv, x.data_ptr())
        print(json.dumps({"case": label + ("-cold" if cold else ""), "op": op, "dtype": dtype, "dims": dims, "levels": lv,
                          "ms_median": med, "ms_min": ms[0], "bytes": byts,
                          "GBps": byts / med / 1e6, "frac_of_peak": byts / med / 1e6 / peak(),
                          "elements_per_s": n / med * 1e3, "plan": plan}), flush=True)


def run_xform(name, reps, timed):
    """mc-pi-<samples log2> (fp32 pairs, disk count) or dot-rows (fp32 rows of 4096)."""
    if name.startswith("mc-pi"):
        n = 1 << int(name.split("-")[2]) if name.count("-") == 2 else 1 << 29
        xf, dtype, dims, lv, byts = "disk", "fp32", (n, 1, 1), "gv", 8 * n
    else:
        xf, dtype, dims, lv = "dot", "fp32", (1 << 16, 1, 1 << 13), "v"
        byts = 8 * (1 << 29)
    n = dims[0] * dims[1] * dims[2]
    x = tensor(n, dtype) * 2 - 1
    y = tensor(n, dtype) * 2 - 1
    cnt = xr.xr_out_count(dims, lv)
    out = torch.zeros(cnt, dtype=torch.int64 if xf == "disk" else TDT[dtype], device="cuda")
    s = torch.cuda.current_stream()
    for _ in range(3):
        assert xr.xr_transform_reduce(xf, dtype, dims, lv, x.data_ptr(), y.data_ptr(), out.data_ptr(), s.cuda_stream) == 0
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        a.record(s)
        xr.xr_transform_reduce(xf, dtype, dims, lv, x.data_ptr(), y.data_ptr(), out.data_ptr(), s.cuda_stream)
        b.record(s)
    torch.cuda.synchronize()
    if timed:
        ms = sorted(a.elapsed_time(b) for a, b in evs)
        med = ms[len(ms) // 2]
        print(json.dumps({"case": name, "dims": dims, "ms_median": med, "ms_min": ms[0], "bytes": byts,
                          "GBps": byts / med / 1e6, "frac_of_peak": byts / med / 1e6 / peak(),
                          "elements_per_s": n / med * 1e3}), flush=True)


def run_heat(reps, timed, n=8192, case="cfg4-heat"):
    t1 = torch.zeros(n * n, dtype=torch.float64, device="cuda")
    t1[:n] = 1.0
    t2 = t1.clone()
    res = torch.zeros(reps + 3, dtype=torch.float64, device="cuda")
    s = torch.cuda.current_stream()
    xr.xr_heat_run(n, n, 3, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    a_, b_ = t1, t2
    for i, (a, b) in enumerate(evs):
        a.record(s)
        xr.xr_heat_step(n, n, a_.data_ptr(), b_.data_ptr(), res[i:].data_ptr(), s.cuda_stream)
        b.record(s)
        a_, b_ = b_, a_
    torch.cuda.synchronize()
    if timed:
        ms = sorted(a.elapsed_time(b) for a, b in evs)
        med = ms[len(ms) // 2]
        byts = 16 * n * n
        print(json.dumps({"case": case, "dims": [n, n], "ms_median": med, "ms_min": ms[0],
                          "bytes": byts, "GBps": byts / med / 1e6, "frac_of_peak": byts / med / 1e6 / peak(),
                          "points_per_s": n * n / med * 1e3}), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("case", nargs="+")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--time", action="store_true")
    ap.add_argument("--cold", action="store_true", help="flush L2 before every timed call")
    a = ap.parse_args()
    cache = {}
    for name in a.case:
        if name == "cfg4-heat":
            run_heat(a.reps, a.time)
            continue
        if name.startswith("heat-"):  # heat-<n>: an n x n grid (odd n: the shifted-staging path)
            run_heat(a.reps, a.time, int(name.split("-")[1]), name)
            continue
        if name.startswith("mc-pi") or name == "dot-rows":
            run_xform(name, a.reps, a.time)
            continue
        for c in cases(name):
            run_reduce(*c, a.reps, a.time, cache, a.cold)


if __name__ == "__main__":
    main()
