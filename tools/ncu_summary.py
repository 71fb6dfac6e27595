#!/usr/bin/env python3
"""Summarise ncu reports (gpurun_out/ncu/*.ncu-rep) into profiles/.

  python tools/ncu_summary.py TAG [--launches CSV]

Writes profiles/ncu_<TAG>.md (one table row per captured kernel) and merges
per-launch DRAM traffic into profiles/ncu_traffic.json (read by bench.py).
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
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__occupancy_limit_registers", "occ lim regs"),
    ("launch__occupancy_limit_shared_mem", "occ lim smem"),
    ("smsp__inst_executed.sum", "inst"),
]
# algorithmic bytes per launch for the kdriver cases
ALG = {"fp32sum": 4 * 2**30 + 4, "cfg3col": 4 * 2**30 + 4 * 32768, "cfg3row": 4 * 2**30 + 4 * 32768,
       "heat": 16 * 8192 * 8192, "cfg5v": 4 * 2**27 + 4 * 2**18}
WORKLOAD = {"fp32sum": "fp32-sum"}


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
    reps = sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "ncu", f"*_{tag}.ncu-rep")))
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
    lines = [f"# ncu summary — {tag}", "",
             "`ncu --set full --clock-control none --import-source on -k regex:<kernel> -s 3 -c 1` "
             "on `tools/kdriver.py <case>` (one B200, cold L2 per replay). Algorithmic bytes from "
             "DESIGN.md section 5.", "",
             "| case | kernel | time (us) | DRAM read | DRAM write | traffic / algorithmic | DRAM TB/s | regs | grid | occ lim (regs/smem) | warps active % |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    for rep in reps:
        case = os.path.basename(rep).rsplit("_", 1)[0]
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
        alg = ALG.get(case)
        ratio = f"{(rd + wr) / alg:.4f}" if alg else "-"
        bw = to_bytes(*d["dram__bytes.sum.per_second"]) / 1e12
        lines.append(f"| {case} | `{kname[:60]}` | {t_us:.1f} | {rd/1e9:.4f} GB | {wr/1e6:.2f} MB | {ratio} | "
                     f"{bw:.2f} | {d['launch__registers_per_thread'][0]} | {d['launch__grid_size'][0]} | "
                     f"{float(d.get('launch__occupancy_limit_registers', ('0',))[0]):.0f}/{float(d.get('launch__occupancy_limit_shared_mem', ('0',))[0]):.0f} | "
                     f"{float(d['sm__warps_active.avg.pct_of_peak_sustained_active'][0]):.1f} |")
        if case in WORKLOAD:
            traffic[WORKLOAD[case]] = rd + wr
        traffic[f"{case}@{tag}"] = rd + wr
    if len(sys.argv) > 3 and sys.argv[2] == "--launches":
        src = sys.argv[3]
        dst = os.path.join(ROOT, "profiles", f"launches_{tag}.csv")
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
    with open(os.path.join(ROOT, "profiles", f"ncu_{tag}.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    json.dump(traffic, open(tpath, "w"), indent=1, sort_keys=True)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
