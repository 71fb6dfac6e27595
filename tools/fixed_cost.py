#!/usr/bin/env python3
"""Fixed per-launch cost: time the R-shape stream reduction (fp32 '+', gwv)
and the heat sweep over a range of sizes and fit t(n) = a + bytes / BW by
least squares; a = launch + ramp + tail, BW = the streaming rate.  One JSON
line per series."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402


def timeit(fn, reps=25):
    s = torch.cuda.current_stream()
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in ev:
        a.record(s)
        fn()
        b.record(s)
    torch.cuda.synchronize()
    return sorted(a.elapsed_time(b) for a, b in ev)[reps // 2] * 1e3  # us


def timeit_b2b(fn, reps=25):
    """Per-launch time of `reps` back-to-back launches with NO event records
    between them (events only around the loop): a launch's drain can overlap
    the next one's start (programmatic dependent launch)."""
    s = torch.cuda.current_stream()
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / reps


def fit(xs, ts):
    A = np.vstack([np.ones(len(xs)), np.array(xs, float)]).T
    (a, b), *_ = np.linalg.lstsq(A, np.array(ts), rcond=None)
    return a, 1.0 / b / 1e3  # us, GB/s (bytes / us -> /1e3 GB/s)


big = torch.rand(1 << 30, device="cuda")
out = torch.zeros(1, device="cuda")
sh = torch.cuda.current_stream().cuda_stream
label = os.environ.get("LABEL", "")
for name, sizes in [("stream-R-fp32", [1 << k for k in range(24, 31)])]:
    xs, ts = [], []
    for n in sizes:
        t = timeit(lambda: xr.xr_reduce("+", "fp32", (n, 1, 1), "gwv", big.data_ptr(), out.data_ptr(), sh))
        xs.append(4 * n)
        ts.append(t)
    a, bw = fit(xs[2:], ts[2:])  # >= 64 MiB (past L2)
    print(json.dumps({"series": name, "label": label, "sizes_bytes": xs, "us": [round(t, 2) for t in ts],
                      "fixed_us": round(a, 2), "stream_GBps": round(bw, 1)}), flush=True)
    ts = [timeit_b2b(lambda: xr.xr_reduce("+", "fp32", (n, 1, 1), "gwv", big.data_ptr(), out.data_ptr(), sh))
          for n in sizes]
    a, bw = fit(xs[2:], ts[2:])
    print(json.dumps({"series": name + "-back-to-back", "label": label, "sizes_bytes": xs,
                      "us": [round(t, 2) for t in ts], "fixed_us": round(a, 2), "stream_GBps": round(bw, 1)}),
          flush=True)
# reference series: torch's own copy (the MEASURED_PEAKS kernel) and torch.sum
for name, mk in [("torch-copy", lambda n: (lambda d=torch.empty(n, device="cuda"): d.copy_(big[:n]))),
                 ("torch-sum", lambda n: (lambda: torch.sum(big[:n])))]:
    xs, ts = [], []
    for n in [1 << k for k in range(24, 30 if name == "torch-copy" else 31)]:
        fn = mk(n)
        ts.append(timeit(fn))
        xs.append((8 if name == "torch-copy" else 4) * n)
    a, bw = fit(xs[2:], ts[2:])
    print(json.dumps({"series": name, "label": label, "sizes_bytes": xs, "us": [round(t, 2) for t in ts],
                      "fixed_us": round(a, 2), "stream_GBps": round(bw, 1)}), flush=True)
del big
xs, ts = [], []
for n in (4096, 5793, 8192, 11585):
    t1 = torch.zeros(n * n, dtype=torch.float64, device="cuda")
    t1[:n] = 1.0
    t2 = t1.clone()
    res = torch.zeros(1, dtype=torch.float64, device="cuda")
    t = timeit(lambda: xr.xr_heat_step(n, n, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), sh))
    xs.append(16 * n * n)
    ts.append(t)
    del t1, t2
a, bw = fit(xs, ts)
print(json.dumps({"series": "heat-fp64", "label": label, "sizes_bytes": xs, "us": [round(t, 2) for t in ts],
                  "fixed_us": round(a, 2), "stream_GBps": round(bw, 1)}), flush=True)
