#!/usr/bin/env python3
"""Host-side cost per xr_reduce call (cfg1 nest, launch bound): wall time per
call of N back-to-back calls (GPU work queued), the pure-host planner
(xr_plan_describe), a bare ctypes call (xr_out_count), and torch's own
smallest launch for reference.  Prints one JSON line."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

N = 20000
dims = (64, 64, 128)
x = torch.randint(-1000, 1000, (64 * 64 * 128,), dtype=torch.int32, device="cuda")
out = torch.zeros(64 * 128, dtype=torch.int32, device="cuda")
s = torch.cuda.current_stream()
sh = s.cuda_stream
res = {}
for lv in ("g", "gwv"):
    for _ in range(100):
        xr.xr_reduce("+", "int32", dims, lv, x.data_ptr(), out.data_ptr(), sh)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(N):
        xr.xr_reduce("+", "int32", dims, lv, x.data_ptr(), out.data_ptr(), sh)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    res[f"xr_reduce_{lv}_host_us"] = (t1 - t0) / N * 1e6
    res[f"xr_reduce_{lv}_total_us"] = (t2 - t0) / N * 1e6
# raw ctypes entry (no Python marshalling helpers)
L = xr._lib
d = xr._dims(dims)
m = xr.mask_of("g")
t0 = time.perf_counter()
for _ in range(N):
    L.xr_reduce(0, 0, d, m, x.data_ptr(), out.data_ptr(), sh)
t1 = time.perf_counter()
torch.cuda.synchronize()
t2 = time.perf_counter()
res["raw_ctypes_g_host_us"] = (t1 - t0) / N * 1e6
res["raw_ctypes_g_total_us"] = (t2 - t0) / N * 1e6
t0 = time.perf_counter()
for _ in range(N):
    xr.xr_plan_describe("+", "int32", dims, "g", x.data_ptr())
res["plan_describe_us"] = (time.perf_counter() - t0) / N * 1e6
t0 = time.perf_counter()
for _ in range(N):
    L.xr_out_count(d, m, None)
res["ctypes_out_count_us"] = (time.perf_counter() - t0) / N * 1e6
y = torch.zeros(1, device="cuda")
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(N):
    y.add_(1.0)
t1 = time.perf_counter()
torch.cuda.synchronize()
res["torch_add_host_us"] = (t1 - t0) / N * 1e6
res["torch_add_total_us"] = (time.perf_counter() - t0) / N * 1e6
print(json.dumps({k: round(v, 3) for k, v in res.items()}))
