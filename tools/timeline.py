#!/usr/bin/env python3
"""Per-CTA timeline of one stream_kernel launch (xr_debug_timeline), to see
where a launch's fixed cost goes (VERDICT r1 "measure first").

  python tools/timeline.py [--elements N ...] [--dtype fp32] [--reps R] [--out FILE]

For each size: R back-to-back launches timed with CUDA events, then one launch
with the timeline on.  Prints one JSON line per size: event time, the
%globaltimer span from the first CTA start to the output write, the spread of
CTA starts, of consumer ends (the tail), the last-CTA fold, and units per CTA.
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

EV = {0: "start", 1: "unit", 2: "unit_done", 3: "cons_end", 4: "fold", 5: "end"}


def q(a, ps=(0, 10, 50, 90, 100)):
    a = np.asarray(a, dtype=np.float64)
    return {f"p{p}": round(float(np.percentile(a, p)), 3) for p in ps} if a.size else {}


def run(n, dtype, op, reps, nest=None, mask="gwv"):
    tdt = {"fp32": torch.float32, "int64": torch.int64, "fp64": torch.float64, "int32": torch.int32}[dtype]
    nest = tuple(nest) if nest else (n, 1, 1)
    n = int(np.prod(nest))
    x = torch.ones(n, dtype=tdt, device="cuda")
    out = torch.zeros(max(1, xr.xr_out_count(nest, mask)), dtype=tdt, device="cuda")
    s = torch.cuda.current_stream()
    for _ in range(3):
        assert xr.xr_reduce(op, dtype, nest, mask, x.data_ptr(), out.data_ptr(), s.cuda_stream) == 0
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        a.record(s)
        xr.xr_reduce(op, dtype, nest, mask, x.data_ptr(), out.data_ptr(), s.cuda_stream)
        b.record(s)
    torch.cuda.synchronize()
    ms = sorted(a.elapsed_time(b) for a, b in evs)
    cap = 1 << 20
    buf = torch.zeros(2 + 2 * cap, dtype=torch.int64, device="cuda")
    buf[1] = cap
    spans = []
    recs_last = None
    for _ in range(3):
        buf[0] = 0
        xr._lib.xr_debug_timeline(buf.data_ptr(), cap)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        xr.xr_reduce(op, dtype, nest, mask, x.data_ptr(), out.data_ptr(), s.cuda_stream)
        b.record(s)
        xr._lib.xr_debug_timeline(None, 0)
        torch.cuda.synchronize()
        cnt = int(buf[0].item())
        r = buf[2:2 + 2 * min(cnt, cap)].cpu().numpy().astype(np.uint64).reshape(-1, 2)
        recs_last = (r, a.elapsed_time(b))
    r, ev_ms = recs_last
    cta = (r[:, 0] >> np.uint64(40)).astype(np.int64)
    ev = ((r[:, 0] >> np.uint64(32)) & np.uint64(0xff)).astype(np.int64)
    unit = (r[:, 0] & np.uint64(0xffffffff)).astype(np.int64)
    t = r[:, 1].astype(np.int64)
    if not (ev == 0).any():
        return {"elements": n, "nest": list(nest), "mask": mask, "dtype": dtype,
                "event_ms_median": ms[len(ms) // 2], "timeline": "none (kernel not instrumented)"}
    t0 = t[ev == 0].min()
    us = (t - t0) / 1e3
    starts = us[ev == 0]
    cons_end = us[ev == 3]
    fold = us[ev == 4]
    end = us[ev == 5]
    units_per_cta = np.bincount(cta[ev == 1], minlength=cta.max() + 1)
    # time between consecutive unit_done records of the same CTA (unit duration in the steady state)
    ud = []
    for c in np.unique(cta):
        tt = np.sort(us[(cta == c) & (ev == 2)])
        ud += list(np.diff(tt))
    plan = xr.xr_plan_describe(op, dtype, nest, mask, x.data_ptr())
    bytes_ = n * x.element_size()
    span = float(end.max()) if end.size else float(cons_end.max())
    return {
        "elements": n, "nest": list(nest), "mask": mask, "dtype": dtype, "bytes": bytes_, "plan": {k: plan[k] for k in ("kernel", "units", "grid")},
        "event_ms_median": ms[len(ms) // 2], "event_ms_min": ms[0],
        "timeline_event_ms": ev_ms,
        "span_us_first_start_to_out": span,
        "launch_overhead_us_event_minus_span": ms[len(ms) // 2] * 1e3 - span,
        "ideal_us_at_7.4TBps": bytes_ / 7.4e12 * 1e6,
        "cta_start_us": q(starts),
        "cons_end_us": q(cons_end),
        "tail_us_last_minus_median_cons_end": float(cons_end.max() - np.median(cons_end)),
        "fold_us": float(end.max() - fold.max()) if fold.size and end.size else None,
        "units_per_cta": q(units_per_cta),
        "unit_us": q(ud),
        "records": int(len(r)),
        "last_real_claim_us": float(us[(ev == 1) & (unit < int(plan["units"]))].max()),
        "unit_done_last_us": float(us[ev == 2].max()) if (ev == 2).any() else None,
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--elements", type=int, nargs="+", default=[1 << 27, 1 << 28, 1 << 30])
    ap.add_argument("--dtype", default="fp32")
    ap.add_argument("--op", default="+")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--out", default=None)
    ap.add_argument("--nest", type=int, nargs=3, default=None, help="3-level nest (overrides --elements)")
    ap.add_argument("--mask", default="gwv")
    a = ap.parse_args()
    lines = []
    for n in ([0] if a.nest else a.elements):
        d = run(n, a.dtype, a.op, a.reps, a.nest, a.mask)
        lines.append(json.dumps(d))
        print(lines[-1], flush=True)
    if a.out:
        with open(a.out, "w") as f:
            f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
