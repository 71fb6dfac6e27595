#!/usr/bin/env python3
"""A/B on one B200: xr_reduce (single pass, warp tiers, TMA staging) vs the
paper's own scheme (xr_reduce_paper: Kepler launch, smem log-step, partial
buffer + second launch).  Prints one JSON line per (shape, mask, dtype, op).

  python tools/ab_paper.py [--reps R]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

TDT = {"int32": torch.int32, "fp32": torch.float32, "fp64": torch.float64}
SZ = {"int32": 4, "fp32": 4, "fp64": 8}
# (label, dims, levels): cfg1; the paper's testsuite sizes (reading C15: the
# reduced loop 2^20, the other two 2 and 32, outer -> inner); 512^3
CASES = [("cfg1", (64, 64, 128), lv) for lv in ("g", "w", "v", "gw", "wv", "gwv")] + [
    ("paper-1M", (1 << 20, 2, 32), "g"), ("paper-1M", (2, 1 << 20, 32), "w"),
    ("paper-1M", (2, 32, 1 << 20), "v"), ("paper-1M", (1 << 20, 2, 32), "gwv")] + [
    ("paper-1M", (1 << 20, 2, 32), "gw"), ("paper-1M", (2, 1 << 20, 32), "wv")] + [
    ("512^3", (512, 512, 512), lv) for lv in ("g", "w", "v", "gw", "wv", "gwv")]
LAUNCHES = {"paper192": (192, 8, 128), "b200": (148 * 8, 8, 128)}


def timeit(fn, reps):
    s = torch.cuda.current_stream()
    for _ in range(3):
        assert fn() == 0
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in ev:
        a.record(s)
        fn()
        b.record(s)
    torch.cuda.synchronize()
    ms = sorted(a.elapsed_time(b) for a, b in ev)
    return ms[len(ms) // 2]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=9)
    args = ap.parse_args()
    for label, dims, lv in CASES:
        for dtype in ("int32", "fp32", "fp64"):
            n = dims[0] * dims[1] * dims[2]
            x = (torch.rand(n, device="cuda") * 10).to(TDT[dtype])
            cnt = xr.xr_out_count(dims, lv)
            out = torch.zeros(cnt, dtype=TDT[dtype], device="cuda")
            sh = torch.cuda.current_stream().cuda_stream
            res = {"case": label, "dims": dims, "levels": lv, "dtype": dtype, "op": "+"}
            res["xreduce_ms"] = timeit(lambda: xr.xr_reduce("+", dtype, dims, lv, x.data_ptr(), out.data_ptr(), sh),
                                       args.reps)
            ref = out.clone()
            for name, (g, w, v) in LAUNCHES.items():
                res[name + "_ms"] = timeit(lambda: xr.xr_reduce_paper("+", dtype, dims, lv, x.data_ptr(), out.data_ptr(),
                                                                      g, w, v, sh), args.reps)
                if dtype == "int32":
                    res[name + "_equal"] = bool(torch.equal(out, ref))
            byts = (n + cnt) * SZ[dtype]
            res["bytes"] = byts
            res["xreduce_GBps"] = byts / res["xreduce_ms"] / 1e6
            res["speedup_vs_paper192"] = res["paper192_ms"] / res["xreduce_ms"]
            res["speedup_vs_b200launch"] = res["b200_ms"] / res["xreduce_ms"]
            print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
