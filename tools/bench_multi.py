#!/usr/bin/env python3
"""N2 measurement: xr_reduce_multi / xr_reduce_multi_at (one launch) vs one
xr_reduce per variable; the A7b rows give every variable its own levels."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

VARS = [("+", "int32"), ("+", "fp64"), ("max", "fp32"), ("^", "int64"), ("&&", "fp32"), ("*", "int32"),
        ("min", "int64"), ("+", "fp32")]
TDT = {"int32": torch.int32, "int64": torch.int64, "fp32": torch.float32, "fp64": torch.float64}


def timeit(fn, reps=21):
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
    return a.elapsed_time(b) / reps


LEVELS_AT = ["v", "w", "g", "wv", "gw", "gv", "gwv", "w"]   # A7b: one mask per variable

for dims, lv in [((64, 64, 128), "v"), ((64, 64, 128), "gwv"), ((4096, 1, 4096), "v"), ((1 << 24, 1, 1), "gwv"),
                 ((64, 64, 128), "g"), ((1, 4096, 4096), "w"), ((64, 64, 128), "at"), ((256, 256, 256), "at")]:
    n = dims[0] * dims[1] * dims[2]
    xs = [(torch.rand(n, device="cuda") * 100).to(TDT[dt]) for _, dt in VARS]
    lvs = LEVELS_AT if lv == "at" else [lv] * len(VARS)
    outs = [torch.zeros(max(1, xr.xr_out_count(dims, m)), dtype=TDT[dt], device="cuda")
            for (_, dt), m in zip(VARS, lvs)]
    sh = torch.cuda.current_stream().cuda_stream
    spec = [(op, dt, m, x.data_ptr(), o.data_ptr()) for (op, dt), m, x, o in zip(VARS, lvs, xs, outs)]
    if lv == "at":
        t_multi = timeit(lambda: xr.xr_reduce_multi_at(spec, dims, sh))
    else:
        t_multi = timeit(lambda: xr.xr_reduce_multi([(op, dt, i, o) for op, dt, _, i, o in spec], dims, lv, sh))
    t_sep = timeit(lambda: [xr.xr_reduce(op, dt, dims, m, i, o, sh) for op, dt, m, i, o in spec])
    byts = sum(x.numel() * x.element_size() for x in xs)
    print(json.dumps({"dims": dims, "levels": lv if lv != "at" else lvs, "vars": len(VARS), "multi_ms": t_multi, "separate_ms": t_sep,
                      "speedup": t_sep / t_multi, "multi_GBps": byts / t_multi / 1e6,
                      "separate_GBps": byts / t_sep / 1e6}))
