#!/usr/bin/env python3
"""Context for BASELINE.md: the paper's Table 2 positions x ops x types at the
paper's stated sizes (reading C15: the reduced loop 2^20, the other two 2 and
32 -- outer to inner -- for the single-level rows; the multi-level rows'
sizes are unstated, so the same 2^26-element nest is used with the reduced
loops spanning it), timed on one B200 kernel-only (xr_reduce, device buffers)
and end to end (xr_reduce_host: pinned host input, H2D + reduce + D2H), next
to the paper's OpenUH milliseconds on a K20c.  CONTEXT ONLY, not a target."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

M = 1 << 20
# position: (dims, levels); Table 2 OpenUH ms for (+, *) x (int, float, double) (@45217-46348)
ROWS = {
    "gang": ((M, 2, 32), "g", [(151.27, 142.99, 244.61), (156.01, 249.27, 254.90)]),
    "worker": ((2, M, 32), "w", [(399.25, 401.33, 610.61), (413.35, 414.50, 664.87)]),
    "vector": ((2, 32, M), "v", [(268.47, 274.06, 532.01), (269.80, 284.68, 529.37)]),
    "gang worker": ((1024, 1024, 64), "gw", [(107.49, 115.10, 212.31), (113.36, 104.44, 223.30)]),
    "worker vector": ((64, 1024, 1024), "wv", [(50.58, 54.85, 107.75), (51.20, 52.75, 105.97)]),
    "gang worker vector": ((256, 512, 512), "gwv", [(8.77, 7.66, 7.65), (8.15, 5.61, 4.87)]),
    "same line gang worker vector": ((1 << 26, 1, 1), "gwv", [(7.55, 7.57, 11.24), (7.25, 7.86, 11.90)]),
}
TYPES = [("int32", torch.int32), ("fp32", torch.float32), ("fp64", torch.float64)]


def dev_time(fn, reps=11):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


for pos, (dims, lv, paper) in ROWS.items():
    n = dims[0] * dims[1] * dims[2]
    for oi, op in enumerate(["+", "*"]):
        for ti, (dt, tdt) in enumerate(TYPES):
            x = (torch.rand(n, device="cuda") * 2).to(tdt) if op == "+" else torch.ones(n, dtype=tdt, device="cuda")
            cnt = xr.xr_out_count(dims, lv)
            out = torch.zeros(cnt, dtype=tdt, device="cuda")
            k_ms = dev_time(lambda: xr.xr_reduce(op, dt, dims, lv, x.data_ptr(), out.data_ptr()))
            host = x.cpu().pin_memory()
            hout = torch.zeros(cnt, dtype=tdt).pin_memory()
            xr.xr_reduce_host(op, dt, dims, lv, host.data_ptr(), hout.data_ptr())
            t0 = time.perf_counter()
            for _ in range(3):
                assert xr.xr_reduce_host(op, dt, dims, lv, host.data_ptr(), hout.data_ptr()) == 0
            e_ms = (time.perf_counter() - t0) / 3 * 1e3
            print(json.dumps({"position": pos, "op": op, "dtype": dt, "dims": dims, "levels": lv,
                              "paper_openuh_ms_k20c": paper[oi][ti], "kernel_ms": k_ms, "e2e_ms": e_ms,
                              "bytes": n * x.element_size()}), flush=True)
