#!/usr/bin/env python3
"""Launch-bound latency: xr_reduce on the cfg1 nest called eagerly vs replayed from a CUDA graph."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

dims = (64, 64, 128)
x = torch.randint(-1000, 1000, (64 * 64 * 128,), dtype=torch.int32, device="cuda")
s = torch.cuda.Stream()
for lv in ["g", "w", "v", "gw", "gv", "wv", "gwv"]:
    o = torch.zeros(xr.xr_out_count(dims, lv), dtype=torch.int32, device="cuda")
    with torch.cuda.stream(s):
        xr.xr_reserve("+", "int32", dims, lv, s.cuda_stream)
        for _ in range(10):
            xr.xr_reduce("+", "int32", dims, lv, x.data_ptr(), o.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
    N = 200
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        a.record()
        for _ in range(N):
            xr.xr_reduce("+", "int32", dims, lv, x.data_ptr(), o.data_ptr(), s.cuda_stream)
        b.record()
    torch.cuda.synchronize()
    eager_us = a.elapsed_time(b) / N * 1e3
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(N):
            xr.xr_reduce("+", "int32", dims, lv, x.data_ptr(), o.data_ptr(), s.cuda_stream)
    g.replay()
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        a.record()
        g.replay()
        b.record()
    torch.cuda.synchronize()
    graph_us = a.elapsed_time(b) / N * 1e3
    print(json.dumps({"case": f"cfg1-{lv}", "eager_us_per_call": eager_us, "graph_us_per_call": graph_us,
                      "bytes": 64 * 64 * 128 * 4, "graph_GBps": 64 * 64 * 128 * 4 / graph_us / 1e3}))
