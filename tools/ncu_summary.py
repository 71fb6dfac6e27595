#!/usr/bin/env python3
"""Summarise ncu reports (gpurun_out/ncu/<case>_<TAG>.ncu-rep) into profiles/.

  python tools/ncu_summary.py TAG [--launches CSV] [--outdir DIR]

<case> is a tools/kdriver.py case name (cfg2-f32-sum, cfg3-col, cfg4-heat,
cfg5-<op>-<dtype>-<mask>, nest-..., mc-pi-N, ...).  Writes
profiles/ncu_<TAG>.md (one row per captured kernel, with ncu's
dram__throughput.avg.pct_of_peak_sustained_elapsed -- the BASELINE metric's
"% of B200 HBM peak (ncu)") and merges per-case records into
profiles/ncu_dram.json ({case: {traffic, dram_pct, time_us, alg_bytes,
source}}; bench.py reads its workload's entry), plus DRAM bytes into
profiles/ncu_traffic.json (history).
"""
import csv
import glob
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__bytes.sum.per_second", "DRAM B/s"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % peak"),
    ("dram__cycles_active.avg.pct_of_peak_sustained_elapsed", "DRAM cycles active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__occupancy_limit_registers", "occ lim regs"),
    ("launch__occupancy_limit_shared_mem", "occ lim smem"),
    ("smsp__inst_executed.sum", "inst"),
]
SIZE = {"int32": 4, "int64": 8, "fp32": 4, "fp64": 8, "f32": 4, "f64": 8, "i32": 4, "i64": 8}
# bench.py workload names of the cfg2 captures
WORKLOAD = {"cfg2-f32-sum": "fp32-sum", "cfg2-f32-max": "fp32-max", "cfg2-f32-min": "fp32-min",
            "cfg2-i64-sum": "int64-sum", "cfg2-i64-max": "int64-max", "cfg2-i64-min": "int64-min",
            "fp32sum": "fp32-sum"}


def out_count(dims, lv):
    c = 1
    for d, ch in enumerate("gwv"):
        if ch not in lv:
            c *= dims[d]
    return c


def alg_bytes(case):
    """Algorithmic bytes per launch of a kdriver case."""
    if case.startswith("cfg2-"):
        return (2**30 + 1) * SIZE[case.split("-")[1]]
    if case in ("cfg3-row", "cfg3-col", "cfg3row", "cfg3col"):
        return 4 * 2**30 + 4 * 32768
    if case in ("cfg4-heat", "heat"):
        return 16 * 8192 * 8192
    if case.startswith("heat-"):
        n = int(case.split("-")[1])
        return 16 * n * n
    if case == "fp32sum":
        return 4 * 2**30 + 4
    if case.startswith("cfg5-"):
        _, _, dt, lv = case.split("-")
        return (2**27 + out_count((512, 512, 512), lv)) * SIZE[dt]
    if case.startswith("nest-"):
        _, _, dt, dims, lv = case.split("-")
        d = tuple(int(v) for v in dims.split("x"))
        return (d[0] * d[1] * d[2] + out_count(d, lv)) * SIZE[dt]
    if case.startswith("mc-pi"):
        return 8 * (1 << int(case.split("-")[2]))
    return None


def to_bytes(v, unit):
    f = float(v.replace(",", ""))
    unit = unit.replace("/second", "").replace("/s", "")
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return None
    return rows[0], rows[1], rows[2]


def main():
    tag = sys.argv[1]
    # --outdir D: write the summary and the merged json files to D instead of
    # profiles/ (used ON the GPU box, where the .ncu-rep files are too large
    # to bring back; the caller copies D into profiles/)
    outdir = os.path.join(ROOT, "profiles")
    if "--outdir" in sys.argv:
        outdir = sys.argv[sys.argv.index("--outdir") + 1]
        for f in ("ncu_traffic.json", "ncu_dram.json"):
            src = os.path.join(ROOT, "profiles", f)
            if os.path.exists(src) and not os.path.exists(os.path.join(outdir, f)):
                os.makedirs(outdir, exist_ok=True)
                with open(src) as a, open(os.path.join(outdir, f), "w") as b:
                    b.write(a.read())
    reps = sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "ncu", f"*_{tag}.ncu-rep")))
    os.makedirs(outdir, exist_ok=True)
    tpath = os.path.join(outdir, "ncu_traffic.json")
    dpath = os.path.join(outdir, "ncu_dram.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
    dram = json.load(open(dpath)) if os.path.exists(dpath) else {}
    lines = [f"# ncu summary — {tag}", "",
             "`ncu --set full --clock-control none --import-source on -k regex:<kernel> -s 3 -c 1` "
             "on `tools/kdriver.py <case>` (one B200, cold L2 per replay). **DRAM %** is "
             "`dram__throughput.avg.pct_of_peak_sustained_elapsed`, the BASELINE metric's "
             "\"% of B200 HBM peak (ncu)\". Algorithmic bytes from DESIGN.md section 5.", "",
             "| case | kernel | time (us) | DRAM % | DRAM read | DRAM write | traffic / algorithmic | DRAM TB/s | "
             "regs | grid | occ lim (regs/smem) | warps active % |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for rep in reps:
        case = os.path.basename(rep)[:-len(f"_{tag}.ncu-rep")]
        r = raw(rep)
        if r is None:
            continue
        hdr, units, vals = r
        d = {m: (vals[hdr.index(m)], units[hdr.index(m)]) for m, _ in METRICS if m in hdr}
        kname = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        rd = to_bytes(*d["dram__bytes_read.sum"])
        wr = to_bytes(*d["dram__bytes_write.sum"])
        t_us = float(d["gpu__time_duration.sum"][0].replace(",", ""))
        if d["gpu__time_duration.sum"][1] == "ms":
            t_us *= 1e3
        elif d["gpu__time_duration.sum"][1] == "ns":
            t_us /= 1e3
        # ncu's "DRAM Throughput" (GPU Speed Of Light section); --set full
        # stores it as dram__cycles_active.avg.pct_of_peak_sustained_elapsed
        pct = None
        for m in ("dram__throughput.avg.pct_of_peak_sustained_elapsed",
                  "dram__cycles_active.avg.pct_of_peak_sustained_elapsed"):
            if m in hdr and vals[hdr.index(m)].strip():
                pct = float(vals[hdr.index(m)].replace(",", ""))
                break
        alg = alg_bytes(case)
        ratio = f"{(rd + wr) / alg:.4f}" if alg else "-"
        bw = to_bytes(*d["dram__bytes.sum.per_second"]) / 1e12 if "dram__bytes.sum.per_second" in d else \
            (rd + wr) / (t_us * 1e-6) / 1e12
        g = lambda m: d.get(m, ("-",))[0]  # noqa: E731  (metrics-only captures lack the launch stats)
        lines.append(f"| {case} | `{kname[:60]}` | {t_us:.1f} | **{pct if pct is None else round(pct, 1)}** | {rd/1e9:.4f} GB | {wr/1e6:.2f} MB | "
                     f"{ratio} | {bw:.2f} | {g('launch__registers_per_thread')} | {g('launch__grid_size')} | "
                     f"{g('launch__occupancy_limit_registers')}/{g('launch__occupancy_limit_shared_mem')} | "
                     f"{g('sm__warps_active.avg.pct_of_peak_sustained_active')} |")
        rec = {"traffic": rd + wr, "dram_pct": pct, "time_us": t_us, "alg_bytes": alg, "kernel": kname,
               "source": f"profiles/ncu_{tag}.md ({os.path.basename(rep)})"}
        dram[f"{case}@{tag}"] = rec
        if case in WORKLOAD:
            dram[WORKLOAD[case]] = rec
            traffic[WORKLOAD[case]] = rd + wr
        traffic[f"{case}@{tag}"] = rd + wr
    if "--launches" in sys.argv:
        src = sys.argv[sys.argv.index("--launches") + 1]
        dst = os.path.join(outdir, f"launches_{tag}.csv")
        with open(src) as f, open(dst, "w") as g:
            g.write("".join(l for l in f if not l.startswith("==")))
        # share of the step per kernel name
        rows = list(csv.DictReader(open(dst)))
        tot = {}
        for r in rows:
            tot[r["Kernel Name"]] = tot.get(r["Kernel Name"], 0) + float(r["Metric Value"].replace(",", ""))
        s = sum(tot.values())
        lines += ["", f"## Launch list (`{os.path.basename(dst)}`: bench.py --steps 5 --warmup 3 under "
                      "`ncu --metrics gpu__time_duration.sum --clock-control none`)", "",
                  "| kernel | launches | total ns | share |", "|---|---|---|---|"]
        for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
            n = sum(1 for r in rows if r["Kernel Name"] == k)
            lines.append(f"| `{k[:70]}` | {n} | {v:.0f} | {v / s:.4f} |")
    with open(os.path.join(outdir, f"ncu_{tag}.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    json.dump(traffic, open(tpath, "w"), indent=1, sort_keys=True)
    json.dump(dram, open(dpath, "w"), indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
