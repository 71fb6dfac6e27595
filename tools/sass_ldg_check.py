#!/usr/bin/env python3
"""Flag kernels whose 16-B global loads are serialized (each LDG.128 consumed
before the next is issued) -- ptxas sometimes sinks the unrolled loads of a
fold loop next to their uses, leaving one or two loads in flight per thread.

  python tools/sass_ldg_check.py [lib.so]   -> per kernel: max batch, #LDG.128

"max batch" = the most LDG.128 issued before the first one's destination
register is read (a window of 40 instructions).  Used by tests/test_sass.py.
"""
import re
import subprocess
import sys

LDG128 = re.compile(r"\bLDG\.E[.A-Z0-9_:]*\.128")
LDS128 = re.compile(r"\bLDS(\.U)?\.128")  # shared-memory stage folds of the ring kernels


def batches(so: str, load=LDG128) -> dict:
    """{demangled kernel name: (max batch, number of 16-B loads)} for kernels with 16-B loads
    (global LDG.128 by default, LDS128 for shared memory)."""
    txt = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True, check=True).stdout
    func = None
    insts = {}
    for line in txt.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            func = m.group(1)
            insts[func] = []
            continue
        m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(.*?);", line)
        if m and func:
            insts[func].append(m.group(1))
    names = subprocess.run(["c++filt"], input="\n".join(insts), capture_output=True, text=True).stdout.splitlines()
    out = {}
    for (f, ins), name in zip(insts.items(), names):
        idx = [i for i, s in enumerate(ins) if load.search(s)]
        if not idx:
            continue
        best = 0
        for i in idx:
            dst = re.search(r"LD[GS]\S*\s+(R\d+)", ins[i]).group(1)
            n = 1
            for s in ins[i + 1:i + 40]:
                parts = s.split(None, 1)
                ops = parts[1] if len(parts) > 1 else ""
                if load.search(s):
                    if re.search(r"\s" + dst + r"\b", s.split(",", 1)[0]):
                        break  # the destination is overwritten by the next load
                    n += 1
                    continue
                if re.search(r"\b" + dst + r"\b", ops):
                    break
            best = max(best, n)
        out[name] = (best, len(idx))
    return out


if __name__ == "__main__":
    so = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_ppopp_xutycc14_b200/libxreduce.so"
    for name, (b, n) in sorted(batches(so).items(), key=lambda kv: kv[1]):
        print(f"{b:2d} {n:3d}  {name}")
