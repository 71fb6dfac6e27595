"""SASS guard (CPU only): the register kernels' fold loops keep >= 4 16-B
loads in flight per thread.  ptxas once sank the unrolled loads of fold_row
next to their uses in some instantiations (2 loads in flight; fp64 && || rows
fell to 0.63 of peak), which no parity test can see -- DESIGN.md section 6."""
import importlib.util
import os
import shutil

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SO = os.path.join(ROOT, "paper_conf_ppopp_xutycc14_b200", "libxreduce.so")


def _checker():
    spec = importlib.util.spec_from_file_location("sass_ldg_check", os.path.join(ROOT, "tools", "sass_ldg_check.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return mod


@pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="cuobjdump not on PATH")
def test_fold_loops_keep_four_loads_in_flight():
    got = _checker().batches(SO)
    fams = ("xr::seg_kernel<", "xr::col_kernel<", "xr::colflat_kernel<")
    checked = {n: b for n, (b, cnt) in got.items() if n.startswith(tuple("void " + f for f in fams)) and cnt >= 4}
    assert len(checked) >= 150, len(checked)  # every (op, dtype, group) instantiation
    bad = {n: b for n, b in checked.items() if b < 4}
    assert not bad, bad


@pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="cuobjdump not on PATH")
def test_ring_stage_folds_keep_four_smem_loads_in_flight():
    """The ring kernels' full-stage folds issue all 4 LDS.128 of a stage before
    the first is consumed (r01: without the fast path and the 3-CTA launch
    bounds, ptxas reused one register quadruple per load -- serialized shared-
    memory latency; 512^3 32-bit && || GWV 0.90 of peak instead of 0.97)."""
    mod = _checker()
    got = mod.batches(SO, mod.LDS128)
    fams = ("xr::stream_kernel<", "xr::rkr_kernel<", "xr::coltma_kernel<")
    checked = {n: b for n, (b, cnt) in got.items() if n.startswith(tuple("void " + f for f in fams))}
    assert len(checked) >= 60, len(checked)
    # no instantiation back to one load at a time; most keep all 4 in flight
    # (fp max/min, whose combine is a compare + select per element, keep 2-3).
    # Exempt: the narrow-row rkr consumers for fp64 max / min, where ptxas
    # issues each stage load next to its compare-select chain at any launch
    # bound (r02; A/B vs the seg kernel they replaced: profiles/ab_rkr_narrow_maxmin_r02bm.jsonl)
    exempt = ("void xr::rkr_kernel<2, double, 4, true>", "void xr::rkr_kernel<3, double, 4, true>")
    bad = {n: b for n, b in checked.items() if b < 2 and not n.startswith(exempt)}
    assert not bad, bad
    assert sum(b >= 4 for b in checked.values()) >= 0.75 * len(checked), sorted(checked.values())


def _sass_by_kernel(so):
    import re
    import subprocess
    txt = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True, check=True).stdout
    func, insts = None, {}
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
    return dict(zip(names, insts.values()))


@pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="cuobjdump not on PATH")
def test_logical_and_folds_use_unsigned_min():
    """`&&` accumulates a nonzero-truth u32 folded by unsigned min (DESIGN.md
    section 5): the 32-bit ring kernels must fold with IMNMX(3).U32 and stay
    within 15 % of the static size of the `+` instantiation (the old 0/1 lift
    cost a compare + select + logic op per element)."""
    k = _sass_by_kernel(SO)
    checked = 0
    for fam in ("xr::stream_kernel<", "xr::rkr_kernel<", "xr::coltma_kernel<"):
        for dt in ("int", "float"):
            land = [n for n in k if n.startswith("void " + fam + "7, " + dt + ",")]
            for n in land:
                add = n.replace(fam + "7, ", fam + "0, ", 1)
                assert any("IMNMX" in s and ".U32" in s for s in k[n]), n
                if add in k:
                    assert len(k[n]) <= 1.15 * len(k[add]), (n, len(k[n]), len(k[add]))
                checked += 1
    assert checked >= 6, checked
