#!/usr/bin/env python3
"""Heat sweep timing for A/B across library builds (XR_LIB_PATH is read at
import, so each build runs in its own process; tools/gpu_*.sh interleaves the
processes).  Per grid: the median of per-launch CUDA-event times and the mean
over `batch` back-to-back sweeps (PDL overlap included).

  XR_LIB_PATH=... python tools/heat_ab.py --tag old --sizes 8192 8191
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="")
    ap.add_argument("--sizes", type=int, nargs="+", default=[8192, 8191, 5793, 11585])
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--batch", type=int, default=30)
    a = ap.parse_args()
    s = torch.cuda.current_stream()
    for n in a.sizes:
        t1 = torch.zeros(n * n, dtype=torch.float64, device="cuda")
        t1[:n] = 1.0
        t2 = t1.clone()
        res = torch.zeros(a.reps + a.batch + 8, dtype=torch.float64, device="cuda")
        xr.xr_heat_run(n, n, 3, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), s.cuda_stream)
        torch.cuda.synchronize()
        bufs = [t1, t2]
        one = []
        for i in range(a.reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            xr.xr_heat_step(n, n, bufs[i & 1].data_ptr(), bufs[(i + 1) & 1].data_ptr(), res[i:].data_ptr(), s.cuda_stream)
            e1.record(s)
            torch.cuda.synchronize()
            one.append(e0.elapsed_time(e1) * 1e3)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for i in range(a.batch):
            xr.xr_heat_step(n, n, bufs[i & 1].data_ptr(), bufs[(i + 1) & 1].data_ptr(), res[a.reps + (i % 8):].data_ptr(),
                            s.cuda_stream)
        e1.record(s)
        torch.cuda.synchronize()
        one.sort()
        print(json.dumps({"tag": a.tag, "n": n, "us_event_median": round(one[len(one) // 2], 2),
                          "us_batch_mean": round(e0.elapsed_time(e1) * 1e3 / a.batch, 2),
                          "bytes": 16 * n * n}), flush=True)
        del t1, t2, bufs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
