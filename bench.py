#!/usr/bin/env python3
"""bench.py -- BASELINE.json's metric on its headline single-GPU workload.

Metric: reduced elements/s (and % of B200 HBM peak) at N GPUs vs the CPU oracle.
Workload (N=1, BASELINE.json configs[1], "cfg2"): 1-D whole-array sum of 2^30
fp32 elements U[0,1), reduction at gang+worker+vector.  One step = one
xr_reduce call (the whole hot path: plan, private partials, warp / CTA / last-
CTA combine, init merge).  N>1 (torchrun): the same 2^30-element array is
gang-sharded, rank r owning the contiguous slice r (strong scaling, the
BASELINE cfg2 reading "1 GPU then sharded 2/4/8 GPUs"), and one step =
xr_reduce_sharded (local single-pass kernel + one cross-GPU combine: the fused
NVLink mailbox exchange inside the same kernel, or one NCCL allreduce).
--scaling weak gives every rank its own 2^30-element slice instead.
`--gpus N` without torchrun (WORLD_SIZE unset) re-launches this script under
torch.distributed.run with N ranks; fewer than N visible GPUs is an error
(exit 2), and so is a WORLD_SIZE that differs from --gpus.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
                  [--scaling strong|weak]
                  [--workload fp32-sum|fp32-max|fp32-min|int64-sum|int64-max|int64-min]

Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "reduced elements/s and % of B200 HBM peak (ncu) at 1/2/4/8 GPUs vs CPU oracle"
WORKLOADS = {
    # name: (op, dtype, recipe, bytes/elem)
    "fp32-sum": ("+", "fp32", "u01", 4),
    "fp32-max": ("max", "fp32", "maxmin", 4),
    "fp32-min": ("min", "fp32", "maxmin", 4),
    "int64-sum": ("+", "int64", "ints", 8),
    "int64-max": ("max", "int64", "maxmin", 8),
    "int64-min": ("min", "int64", "maxmin", 8),
}
DTYPE_TAG = {"fp32": "f32", "fp64": "f64", "int32": "i32", "int64": "i64"}
N_PER_GPU = 1 << 30
FALLBACK_HBM_GBS = 6650.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=500)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="xreduce", choices=["xreduce", "reference"])
    ap.add_argument("--workload", default="fp32-sum", choices=sorted(WORKLOADS))
    ap.add_argument("--elements", type=int, default=N_PER_GPU,
                    help="elements of the whole array (strong scaling) or per GPU (weak)")
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="strong (default, BASELINE cfg2: the one 2^30-element array sharded over N GPUs) "
                         "or weak (2^30 elements per GPU)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--force-comm", action="store_true",
                    help="use the NCCL sharded path even at world size 1 (exercises xr_comm_*)")
    return ap.parse_args()


def free_port() -> int:
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def launch_ranks(args):
    """--gpus N > 1 outside torchrun: spawn the N ranks ourselves (one process
    per GPU, NCCL over NVLink).  Returns the exit code, or None to run here."""
    world_env = os.environ.get("WORLD_SIZE")
    if world_env is not None:
        if int(world_env) != args.gpus:
            sys.stderr.write(f"bench.py: WORLD_SIZE={world_env} but --gpus {args.gpus}; launch one rank per GPU "
                             f"(torchrun --nproc-per-node {args.gpus}) or drop --gpus\n")
            return 2
        return None
    if args.gpus <= 1 or args.impl == "reference":
        return None
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} needs {args.gpus} visible GPUs, this host has {have}\n")
        return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def dist_env():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def make_input(wl, n, start, total):
    import datagen
    from datagen import recipes
    op, dtype, kind, _ = WORKLOADS[wl]
    seed = datagen.case_seed(2, {"+": 0, "max": 2, "min": 3}[op], {"fp32": 2, "int64": 1}[dtype], 7)
    if kind == "ints":  # int64 sum: U_int[-2^31, 2^31)
        return datagen.uniform_int(seed, n, -(2**31), 2**31 - 1, np.int64, start)
    return recipes.make(kind, (total, 1, 1), 7, dtype, seed, start=start, n=n)


def workload_desc(wl, n, world, scaling="strong"):
    op, dtype, kind, _ = WORKLOADS[wl]
    return {
        "workload": f"cfg2: 1-D whole-array '{op}' over {n * world} {dtype} elements ({kind}), "
                    f"level_mask gang+worker+vector" + (f", gang-sharded over {world} GPUs ({n} per GPU, "
                                                       f"{scaling} scaling) + one cross-GPU combine"
                                                       if world > 1 else ""),
        "nest_dims_per_gpu": [n, 1, 1],
        "level_mask": "gwv",
        "op": op,
        "elements_per_gpu": n,
        "l2": "input per GPU (%.1f GiB) is larger than L2 (126 MB): no flush needed" % (
            n * WORKLOADS[wl][3] / 2**30),
        "parallelism": f"gang-sharded x{world}" if world > 1 else "single GPU",
    }


# --------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,utilization.gpu,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            out, _ = self.p.communicate(timeout=5)
        except Exception:
            self.p.kill()
            out = ""
        rows = []
        for line in out.strip().splitlines():
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 8:
                rows.append(parts)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"], "samples": 0}
        loaded = [r for r in rows if r[2].isdigit() and int(r[2]) > 0] or rows
        sm = [int(r[0]) for r in loaded if r[0].isdigit()]
        mx = [int(r[1]) for r in rows if r[1].isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in loaded for k in range(4) if r[4 + k].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(loaded)}


def peak_hbm():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_record(wl):
    """The committed ncu capture of this workload's kernel (profiles/ncu_dram.json,
    written by tools/ncu_summary.py): DRAM bytes per launch and
    dram__throughput.avg.pct_of_peak_sustained_elapsed, with its source."""
    p = os.path.join(ROOT, "profiles", "ncu_dram.json")
    try:
        with open(p) as f:
            return json.load(f).get(wl)
    except Exception:
        return None


# --------------------------------------------------------------------- CPU oracle legs
def oracle_rate(wl, x_sample: np.ndarray, seconds: float):
    """The oracle as it stands, single-threaded, on a bounded sample."""
    import oracle
    op, dtype, _, _ = WORKLOADS[wl]
    n = x_sample.size
    reps, t0 = 0, time.perf_counter()
    while True:
        oracle.reduce(op, dtype, (n, 1, 1), "gwv", x_sample)
        reps += 1
        el = time.perf_counter() - t0
        if el >= seconds:
            break
    return reps * n / el, reps, el


def openmp_rate(wl, x_sample: np.ndarray, seconds: float):
    """The all-cores OpenMP CPU baseline (cpubase/) on the same sample."""
    import cpubase
    op, dtype, _, _ = WORKLOADS[wl]
    n = x_sample.size
    cpubase.reduce(op, dtype, (n, 1, 1), "gwv", x_sample)  # spin up the thread pool
    reps, t0 = 0, time.perf_counter()
    while True:
        cpubase.reduce(op, dtype, (n, 1, 1), "gwv", x_sample)
        reps += 1
        el = time.perf_counter() - t0
        if el >= seconds:
            break
    return reps * n / el, reps, el, cpubase.num_procs()


def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    wl = args.workload
    n = args.elements // args.gpus if args.scaling == "strong" else args.elements
    sample_n = min(n, 1 << 24)  # bounded sample per step: the whole run stays within minutes
    x = make_input(wl, sample_n, 0, n)
    per_step = []
    for i in range(args.warmup + args.steps):
        rate, reps, el = oracle_rate(wl, x, 0.0)
        if i >= args.warmup:
            per_step.append(el)
    t = sum(per_step)
    value = args.steps * sample_n / t
    line = {
        "metric": METRIC, "value": value, "unit": "elements/s", "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": DTYPE_TAG[WORKLOADS[wl][1]],
        "data": "synthetic (seeded splitmix64 generator, datagen/)", "impl": "reference",
        "config": workload_desc(wl, n, args.gpus, args.scaling),
        "cpu_baseline": {"value": value, "unit": "elements/s", "cores": 1, "kind": "oracle",
                         "sample": f"first {sample_n} elements of the workload per step (plain C oracle, 1 thread)"},
        "e2e": {"value": value, "unit": "elements/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    emit(line)
    return 0


# --------------------------------------------------------------------- GPU arm
def timed_loop(step, steps, stream, world, per_step=True):
    """K steps bracketed by barrier + synchronize; returns (max-over-ranks ms
    of the whole loop, per-step event ms on this rank).  per_step=False keeps
    event records out of the stream between steps, so back-to-back launches
    can overlap one launch's drain with the next one's start (programmatic
    dependent launch); the per-step list is then empty."""
    import torch
    import torch.distributed as dist
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(steps if per_step else 0)]
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0.record(stream)
    for i in range(steps):
        if per_step:
            ev[i][0].record(stream)
        step()
        if per_step:
            ev[i][1].record(stream)
    t1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    total = t0.elapsed_time(t1)
    if world > 1:
        t = torch.tensor([total], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total = float(t.item())
    return total, [x.elapsed_time(y) for x, y in ev]


def pinned_h2d_gbs(host, dev, reps=3):
    """Measured pinned host -> device copy bandwidth (the e2e ceiling)."""
    import torch
    s = torch.cuda.current_stream()
    best = None
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(s)
        dev.copy_(host, non_blocking=True)
        b.record(s)
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        best = ms if best is None else min(best, ms)
    return host.numel() * host.element_size() / (best / 1e3) / 1e9


def run_gpu(args):
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_xutycc14_b200 as xr

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    use_comm = world > 1 or args.force_comm
    if use_comm:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        os.environ.setdefault("RANK", str(rank))
        os.environ.setdefault("WORLD_SIZE", str(world))
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    wl = args.workload
    op, dtype, kind, esz = WORKLOADS[wl]
    if args.scaling == "strong":  # the whole array is fixed; rank r owns gang slice r
        total = args.elements
        if total % world:
            raise SystemExit(f"--elements {total} is not divisible by {world} GPUs")
        n = total // world
    else:
        n = args.elements
        total = n * world
    tdt = {"fp32": torch.float32, "int64": torch.int64}[dtype]

    # inputs: seeded host generation of this rank's gang slice, pinned, then resident in HBM
    host = torch.from_numpy(make_input(wl, n, rank * n, total)).pin_memory()
    x = host.to("cuda", non_blocking=False)
    out = torch.zeros(1, dtype=tdt, device="cuda")
    stream = torch.cuda.current_stream()
    sh = stream.cuda_stream
    comm = xr.Comm() if use_comm else None
    if use_comm:
        dist.barrier()  # ranks arrive together at the first (fused) exchange

    def local_step():
        st = xr.xr_reduce(op, dtype, (n, 1, 1), "gwv", x.data_ptr(), out.data_ptr(), sh)
        if st != 0:
            raise xr.XReduceError(st, "bench local step")

    def step():
        if comm is None:
            return local_step()
        st = xr._lib.xr_reduce_sharded(xr.OPS[op], xr.DTYPES[dtype], xr._dims((n, 1, 1)), xr.mask_of("gwv"),
                                       x.data_ptr(), out.data_ptr(), comm.handle, sh)
        if st != 0:
            raise xr.XReduceError(st, "bench step")

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    exchange = None
    if comm is not None:
        # the fused exchange (local reduction + NVLink peer mailboxes in ONE
        # kernel) must agree with the NCCL path; otherwise fall back to NCCL
        q = comm.query()
        exchange = "fused NVLink peer-mailbox exchange inside the reduction kernel" if q["fused"] else \
            "ncclAllReduce after the local kernel"
        if q["fused"]:
            step()
            torch.cuda.synchronize()
            fused_val = out.clone()
            comm.set_fused(False)
            step()
            torch.cuda.synchronize()
            nccl_val = out.clone()
            ok = bool(torch.equal(fused_val, nccl_val)) if dtype != "fp32" else \
                bool(torch.allclose(fused_val.double(), nccl_val.double(), rtol=1e-5))
            flag = torch.tensor([1 if (ok and comm.query()["status"] == 0) else 0], device="cuda")
            dist.all_reduce(flag, op=dist.ReduceOp.MIN)
            if int(flag.item()) == 1:
                comm.set_fused(True)  # collective: every rank takes this branch
            else:
                exchange = "ncclAllReduce after the local kernel (fused exchange disagreed or timed out; disabled)"
            for _ in range(3):
                step()
            torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)  # let the sampler attach
    launches0 = xr.xr_launch_count()
    total_ms, _ = timed_loop(step, args.steps, stream, world, per_step=False)
    launches = xr.xr_launch_count() - launches0
    ck = clocks.stop()
    ms_step = total_ms / args.steps
    value = total * args.steps / (total_ms / 1e3)

    # the dominant kernel's average launch duration (roofline.achieved): the
    # local reduction timed alone, one CUDA-event pair per launch (so launches
    # do not overlap); at N>1 this is also the kernel-only time without exchange
    loc_total, per = timed_loop(local_step, args.steps, stream, world)
    kern_ms = statistics.mean(per)
    multi = None
    if use_comm:  # N>1 (or --force-comm at N=1, which exercises the same code)
        # 1-GPU reference time in the same run: rank 0 reduces the whole
        # strong-scaling array (its own slice repeated: timing does not depend
        # on the values) or, weak, its own slice
        t1_ms = None
        if rank == 0:
            if args.scaling == "strong":
                xf = x.repeat(world)
                of = torch.zeros(1, dtype=tdt, device="cuda")

                def full_step():
                    st = xr.xr_reduce(op, dtype, (total, 1, 1), "gwv", xf.data_ptr(), of.data_ptr(), sh)
                    if st != 0:
                        raise xr.XReduceError(st, "bench 1-GPU reference step")
                for _ in range(3):
                    full_step()
                t1_total, _ = timed_loop(full_step, args.steps, stream, 1)
                t1_ms = t1_total / args.steps
                del xf
            else:
                t1_ms = loc_total / args.steps
        peak0, _ = peak_hbm()
        multi = {
            "exchange": exchange,
            "kernel_only_ms_per_step": loc_total / args.steps,
            "kernel_plus_exchange_ms_per_step": ms_step,
            "exchange_ms_per_step": ms_step - loc_total / args.steps,
            "aggregate_elements_per_s": value,
            "aggregate_roofline": {"achieved_gbs": total * esz / (ms_step / 1e3) / 1e9,
                                   "peak_gbs": world * peak0,
                                   "frac": total * esz / (ms_step / 1e3) / 1e9 / (world * peak0)},
            "one_gpu_ms_same_run": t1_ms,
            "efficiency_t1_over_n_tn": (t1_ms / (world * ms_step)) if (t1_ms and args.scaling == "strong")
            else (t1_ms / ms_step if t1_ms else None),
            "timing": "CUDA events on each rank, barrier + synchronize around the loop, max over ranks",
        }
    plan = xr.xr_plan_describe(op, dtype, (n, 1, 1), "gwv", x.data_ptr(), torch.cuda.get_device_properties(local).multi_processor_count)
    kernel_name = {"stream": "stream_kernel (cp.async.bulk smem ring, single pass)",
                   "seg": "seg_kernel", "col": "col_kernel", "coltma": "coltma_kernel"}.get(plan["kernel"], plan["kernel"]) + \
        f" [{plan['shape']} shape, {plan['units']} units, grid {plan['grid']}]"
    peak, peak_src = peak_hbm()
    alg_bytes = n * esz + esz  # read every input element once + write one output
    achieved = alg_bytes / (kern_ms / 1e3) / 1e9
    ncu = ncu_record(wl)

    # e2e through the C ABI with HOST buffers (H2D of the step's input + D2H of the result)
    e2e = None
    if args.e2e_steps > 0:
        out_h = np.zeros(1, dtype={"fp32": np.float32, "int64": np.int64}[dtype])
        hp = host.data_ptr()

        def host_call():
            if comm is None:
                return xr.xr_reduce_host(op, dtype, (n, 1, 1), "gwv", hp, out_h.ctypes.data, sh)
            return xr._lib.xr_reduce_sharded_host(xr.OPS[op], xr.DTYPES[dtype], xr._dims((n, 1, 1)),
                                                  xr.mask_of("gwv"), hp, out_h.ctypes.data, comm.handle, sh)
        assert host_call() == 0  # warm the staging buffers
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            st = host_call()
            assert st == 0, st
        el = time.perf_counter() - t0
        if world > 1:
            t = torch.tensor([el], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            el = float(t.item())
        h2d = pinned_h2d_gbs(host, x)
        e2e = {"value": total * args.e2e_steps / el, "unit": "elements/s",
               "h2d_bytes_per_step": n * esz, "d2h_bytes_per_step": esz, "steps": args.e2e_steps,
               "api": "xr_reduce_host (C ABI: pinned host input, chunked H2D overlapped with the reduction)"
               if world == 1 else "xr_reduce_sharded_host (C ABI: chunked H2D + local reduction + NCCL)",
               "h2d_gbs_achieved": n * esz * args.e2e_steps / el / 1e9,
               "pinned_h2d_gbs_measured": h2d,
               "frac_of_pinned_h2d": n * esz * args.e2e_steps / el / 1e9 / h2d}

    cpu = cpu_omp = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        sample_n = min(n, 1 << 26)
        model = cpu_model()
        rate, reps, el = oracle_rate(wl, host.numpy()[:sample_n], args.cpu_seconds)
        cpu = {"value": rate, "unit": "elements/s", "cores": 1, "kind": "oracle", "cpu_model": model,
               "sample": f"{reps} x oracle over the first {sample_n} elements ({el:.1f} s, 1 thread)"}
        rate, reps, el, cores = openmp_rate(wl, host.numpy()[:sample_n], min(args.cpu_seconds, 3.0))
        cpu_omp = {"value": rate, "unit": "elements/s", "cores": cores, "kind": "openmp", "cpu_model": model,
                   "sample": f"{reps} x cpubase/omp.c over the first {sample_n} elements ({el:.1f} s, "
                             f"{cores} threads)"}

    if rank == 0:
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": ncu.get("traffic") if ncu else None,
                "peak_source": peak_src,
                # the metric's own unit: ncu dram__throughput % of peak for this
                # kernel, from the committed capture named in ncu_source
                "ncu_dram_pct": ncu.get("dram_pct") if ncu else None,
                "ncu_source": ncu.get("source") if ncu else None,
                "kernel": kernel_name,
                "algorithmic_bytes_per_launch": alg_bytes,
                "kernel_ms_mean": kern_ms, "kernel_ms_min": min(per)}
        line = {
            "metric": METRIC, "value": value, "unit": "elements/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": args.scaling,
            "vs_baseline": None, "dtype": DTYPE_TAG[dtype],
            "data": "synthetic (seeded splitmix64 generator, datagen/)",
            "config": dict(workload_desc(wl, n, world, args.scaling), **({"exchange": exchange} if exchange else {})),
            "roofline": roof,
            "hbm_frac_of_peak": achieved / peak,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": ck,
            "cpu_baseline": cpu,
            "cpu_baseline_openmp": cpu_omp,
        }
        if multi is not None:
            line["multi_gpu"] = multi
        emit(line)
    if comm is not None:
        comm.close()
    if use_comm:
        dist.destroy_process_group()
    return 0


_JSON_FD = None


def emit(line: dict):
    """The ONE JSON line, on the process's original stdout.  Everything else
    (NCCL's "NCCL version ..." banner, library prints) was redirected to
    stderr in main(), so the line stays alone on stdout."""
    data = (json.dumps(line) + "\n").encode()
    if _JSON_FD is None:
        sys.stdout.write(data.decode())
        sys.stdout.flush()
    else:
        os.write(_JSON_FD, data)


def main():
    global _JSON_FD
    args = parse()
    rc = launch_ranks(args)
    if rc is not None:
        return rc
    # keep stdout for the JSON line only: fd 1 -> stderr for the rest of the run
    sys.stdout.flush()
    _JSON_FD = os.dup(1)
    os.dup2(2, 1)
    if args.impl == "reference":
        return run_reference(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
