#!/usr/bin/env python3
"""Same-process A/B of planner environment overrides (XR_* variables are read
on every call), interleaved so that box-to-box and drift differences cancel.

  python tools/ab_env.py --cases cfg5-mul-fp64-gw cfg3-col \
      --cfg A: --cfg B:XR_COLTMA_BOX=256 [--rounds 7] [--batch 10]

Cases are tools/kdriver.py names.  Each round runs every config once per case:
`batch` back-to-back launches between two CUDA events (mean per launch; PDL
overlap included, as in a real stream of calls).  Prints one JSON line per
(case, config): median / min over rounds and the ratio to the first config.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

import kdriver  # noqa: E402
import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402


def parse_cfg(spec):
    name, _, rest = spec.partition(":")
    env = {}
    for kv in filter(None, rest.split(",")):
        k, _, v = kv.partition("=")
        env[k] = v
    return name, env


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cases", nargs="+", required=True)
    ap.add_argument("--cfg", action="append", required=True, help="NAME:VAR=VAL,VAR=VAL (NAME: for defaults)")
    ap.add_argument("--rounds", type=int, default=7)
    ap.add_argument("--batch", type=int, default=10)
    ap.add_argument("--single", action="store_true",
                    help="time each launch alone (events around it, synchronised: no overlap with the next launch)")
    a = ap.parse_args()
    cfgs = [parse_cfg(c) for c in a.cfg]
    keys = sorted({k for _, e in cfgs for k in e})
    s = torch.cuda.current_stream()
    for case in a.cases:
        (label, op, dtype, dims, lv), = kdriver.cases(case)
        n = dims[0] * dims[1] * dims[2]
        x = kdriver.tensor(n, dtype)
        out = torch.zeros(xr.xr_out_count(dims, lv), dtype=kdriver.TDT[dtype], device="cuda")
        res = {name: [] for name, _ in cfgs}
        plans = {}

        def setenv(env):
            for k in keys:
                os.environ.pop(k, None)
            os.environ.update(env)

        for name, env in cfgs:  # warm-up (workspace growth, attributes)
            setenv(env)
            plans[name] = xr.xr_plan_describe(op, dtype, dims, lv, x.data_ptr())
            for _ in range(3):
                assert xr.xr_reduce(op, dtype, dims, lv, x.data_ptr(), out.data_ptr(), s.cuda_stream) == 0
        torch.cuda.synchronize()
        for r in range(a.rounds):
            order = cfgs if r % 2 == 0 else cfgs[::-1]
            for name, env in order:
                setenv(env)
                if a.single:
                    ts = []
                    for _ in range(a.batch):
                        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        e0.record(s)
                        st = xr.xr_reduce(op, dtype, dims, lv, x.data_ptr(), out.data_ptr(), s.cuda_stream)
                        assert st == 0, (case, name, xr.xr_strerror(st))
                        e1.record(s)
                        torch.cuda.synchronize()
                        ts.append(e0.elapsed_time(e1) * 1e3)
                    res[name].append(statistics.median(ts))
                    continue
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                for _ in range(a.batch):
                    st = xr.xr_reduce(op, dtype, dims, lv, x.data_ptr(), out.data_ptr(), s.cuda_stream)
                    assert st == 0, (case, name, xr.xr_strerror(st))
                e1.record(s)
                torch.cuda.synchronize()
                res[name].append(e0.elapsed_time(e1) / a.batch * 1e3)
        setenv({})
        base = statistics.median(res[cfgs[0][0]])
        for name, env in cfgs:
            med = statistics.median(res[name])
            p = plans[name]
            print(json.dumps({"case": case, "cfg": name, "env": env, "us_median": round(med, 2),
                              "us_min": round(min(res[name]), 2), "ratio": round(med / base, 4),
                              "plan": {k: p[k] for k in ("kernel", "splits", "units", "grid")}}), flush=True)
        del x, out
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
