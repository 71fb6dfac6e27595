"""CPU-only tests of the C-ABI boundary: the library loads, exports every symbol
include/xreduce.h declares, validates arguments before touching CUDA, and its
host-side planner and shard planner (8(e)) behave."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "xreduce.h")


@pytest.fixture(scope="module")
def xr():
    import paper_conf_ppopp_xutycc14_b200 as m
    return m


def header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(xr_[a-z_0-9]+)\s*\(", src)))


def header_enums():
    src = re.sub(r"/\*.*?\*/", "", open(HEADER).read(), flags=re.S)
    vals = {k: int(v, 0) for k, v in re.findall(r"\b(XR_[A-Z_0-9]+)\s*=\s*(0x[0-9a-fA-F]+|\d+)", src)}
    vals.update({k: int(v.rstrip("u"), 0) for k, v in
                 re.findall(r"#define\s+(XR_[A-Z_]+)\s+(0x[0-9a-fA-F]+u?)", src)})
    return vals


def test_library_exports_every_declared_symbol(xr):
    lib = ctypes.CDLL(xr.LIB_PATH)
    declared = header_functions()
    assert len(declared) >= 16
    for name in declared:
        assert hasattr(lib, name), name
    assert set(declared) == set(xr.EXPORTED)


def test_codes_match_header_and_oracle(xr):
    e = header_enums()
    assert [e[k] for k in ["XR_OP_ADD", "XR_OP_MUL", "XR_OP_MAX", "XR_OP_MIN", "XR_OP_BAND",
                           "XR_OP_BOR", "XR_OP_BXOR", "XR_OP_LAND", "XR_OP_LOR"]] == list(range(9))
    assert [e[k] for k in ["XR_INT32", "XR_INT64", "XR_FP32", "XR_FP64"]] == list(range(4))
    assert (e["XR_GANG"], e["XR_WORKER"], e["XR_VECTOR"], e["XR_INIT_FROM_OUT"]) == (1, 2, 4, 0x100)
    assert xr.OPS == oracle.OPS and xr.DTYPES == oracle.DTYPES
    assert (xr.GANG, xr.WORKER, xr.VECTOR, xr.INIT_FROM_OUT) == \
        (oracle.GANG, oracle.WORKER, oracle.VECTOR, oracle.INIT_FROM_OUT)
    assert (e["XR_OK"], e["XR_ERR_INVALID"], e["XR_ERR_UNSUPPORTED"], e["XR_ERR_CUDA"],
            e["XR_ERR_NCCL"], e["XR_ERR_NOMEM"]) == (0, 1, 2, 3, 4, 5)


def test_strerror(xr):
    for st in range(6):
        assert xr.xr_strerror(st).startswith("XR_")
    assert "unknown" in xr.xr_strerror(99)


@pytest.mark.parametrize("levels", ["g", "w", "v", "gw", "gv", "wv", "gwv"])
@pytest.mark.parametrize("dims", [(64, 64, 128), (4, 0, 3), (1, 1, 1), (7, 1, 9)])
def test_out_count_matches_oracle(xr, dims, levels):
    assert xr.xr_out_count(dims, levels) == oracle.out_count(dims, levels)


def test_validation_without_gpu(xr):
    fake = 0x10000
    d = (2, 2, 2)
    # bitwise on fp -> unsupported (C3), for every mask
    for op in "&|^":
        for dt in ("fp32", "fp64"):
            assert xr.xr_reduce(op, dt, d, 7, fake, fake * 2) == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce("+", "fp32", d, 0, fake, fake * 2) == xr.ERR_INVALID          # no level
    assert xr.xr_reduce("+", "fp32", d, 0x9, fake, fake * 2) == xr.ERR_INVALID        # stray bit
    assert xr.xr_reduce("+", "fp32", (-1, 2, 2), 1, fake, fake * 2) == xr.ERR_INVALID
    assert xr.xr_reduce(9, "fp32", d, 1, fake, fake * 2) == xr.ERR_INVALID
    assert xr.xr_reduce("+", 7, d, 1, fake, fake * 2) == xr.ERR_INVALID
    assert xr.xr_reduce("+", "fp32", d, 1, 0, fake) == xr.ERR_INVALID                 # null in
    assert xr.xr_reduce("+", "fp32", d, 1, fake, 0) == xr.ERR_INVALID                 # null out
    assert xr.xr_reduce("+", "fp32", d, 1, fake + 2, fake * 2) == xr.ERR_INVALID      # misaligned
    assert xr.xr_reduce("+", "fp64", d, 1, fake, fake * 2 + 4) == xr.ERR_INVALID
    assert xr.xr_reduce("+", "fp32", d, 1, fake, fake + 8) == xr.ERR_INVALID          # overlap
    assert xr.xr_reduce("+", "int32", (2**40, 2**30, 1), 1, fake, fake * 2) == xr.ERR_INVALID
    # empty output: valid no-op without any CUDA call
    assert xr.xr_reduce("+", "int32", (4, 0, 3), 1, 0, 0) == xr.OK
    assert xr.xr_reduce_host("+", "int32", (0, 5, 5), 2, 0, 0) == xr.OK


def test_multi_validation_without_gpu(xr):
    """xr_reduce_multi / xr_reduce_multi_at validate every variable before any
    CUDA call (include/xreduce.h): counts, masks, ops, alignment, overlaps."""
    f = 0x100000
    d = (2, 2, 2)
    ok = ("+", "int32", "v", f, f * 4)
    assert xr.xr_reduce_multi_at([], d) == xr.ERR_INVALID
    assert xr.xr_reduce_multi_at([ok] * 9, d) == xr.ERR_INVALID
    assert xr.xr_reduce_multi_at([ok, ("+", "int32", 0, f, f * 5)], d) == xr.ERR_INVALID        # no level
    assert xr.xr_reduce_multi_at([ok, ("+", "int32", 0x11, f, f * 5)], d) == xr.ERR_INVALID     # stray bit
    assert xr.xr_reduce_multi_at([ok, ("^", "fp64", "g", f, f * 5)], d) == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce_multi_at([ok, ("+", "fp64", "g", f, f * 5 + 4)], d) == xr.ERR_INVALID  # misaligned out
    assert xr.xr_reduce_multi_at([ok, ("+", "fp64", "g", 0, f * 5)], d) == xr.ERR_INVALID      # null in
    assert xr.xr_reduce_multi_at([ok, ("+", "int32", "gw", f, f * 4 + 8)], d) == xr.ERR_INVALID  # outputs overlap
    assert xr.xr_reduce_multi_at([ok, ("+", "int32", "g", f * 4, f * 5)], d) == xr.ERR_INVALID  # out over an input
    assert xr.xr_reduce_multi_at([ok], (-1, 2, 2)) == xr.ERR_INVALID
    assert xr.xr_reduce_multi([("+", "int32", f, f * 4)] * 9, d, "g") == xr.ERR_INVALID
    # every output empty: a valid no-op without any CUDA call
    assert xr.xr_reduce_multi_at([("+", "int32", "g", 0, 0), ("max", "fp64", "gv", 0, 0)], (4, 0, 3)) == xr.OK


# ------------------------------------------------------------------ planner (a0)
SHAPE_TABLE = {
    # mask -> canonical shape for a nest with 3 non-unit dims
    "g": ("RK", [64, 8192, 0]), "w": ("KRK", [64, 64, 128]), "v": ("KR", [4096, 128, 0]),
    "gw": ("RK", [4096, 128, 0]), "gv": ("RKR", [64, 64, 128]), "wv": ("KR", [64, 8192, 0]),
    "gwv": ("R", [524288, 0, 0]),
}


@pytest.mark.parametrize("levels", sorted(SHAPE_TABLE))
def test_plan_canonical_shapes_cfg1(xr, levels):
    p = xr.xr_plan_describe("+", "int32", (64, 64, 128), levels, in_addr=256)
    shape, cd = SHAPE_TABLE[levels]
    assert p["shape"] == shape and p["cdims"] == cd
    assert p["out_count"] == oracle.out_count((64, 64, 128), levels)
    assert p["kernel"] in (("col", "coltma", "colflat", "colsmall", "thincol") if shape in ("RK", "KRK")
                           else ("seg", "stream", "rows", "rkr", "shortrow"))


def test_plan_canonical_cfg2_cfg3_cfg5(xr):
    assert xr.xr_plan_describe("+", "fp32", (2**30, 1, 1), "gwv", 256)["shape"] == "R"
    assert xr.xr_plan_describe("+", "fp32", (32768, 1, 32768), "v", 256)["cdims"] == [32768, 32768, 0]
    c = xr.xr_plan_describe("+", "fp32", (1, 32768, 32768), "w", 256)
    assert c["shape"] == "RK" and c["cdims"] == [32768, 32768, 0] and c["vec"] == 4
    assert c["kernel"] == "coltma"
    # {1,R,C}+W and {R,1,C}+G run the same column plan (a0)
    c2 = xr.xr_plan_describe("+", "fp32", (32768, 1, 32768), "g", 256)
    assert {k: c[k] for k in ("shape", "cdims", "splits", "units")} == \
        {k: c2[k] for k in ("shape", "cdims", "splits", "units")}
    for lv, shape in [("g", "RK"), ("w", "KRK"), ("v", "KR"), ("gw", "RK"), ("gv", "RKR"),
                      ("wv", "KR"), ("gwv", "R")]:
        assert xr.xr_plan_describe("*", "int64", (512, 512, 512), lv, 256)["shape"] == shape


def test_plan_edge_cases(xr):
    assert xr.xr_plan_describe("+", "int32", (4, 0, 3), "g", 0)["shape"] == "none"
    f = xr.xr_plan_describe("+", "int32", (4, 0, 3), "w", 0)
    assert f["shape"] == "fill" and f["out_count"] == 12
    assert xr.xr_plan_describe("+", "int32", (1, 1, 1), "gwv", 0)["shape"] == "ident"
    assert xr.xr_plan_describe("+", "int32", (5, 1, 7), "w", 0)["shape"] == "ident"
    # extent-1 toggling changes nothing (P11 at the planner level)
    a = xr.xr_plan_describe("max", "fp64", (9, 1, 33), "v", 0)
    b = xr.xr_plan_describe("max", "fp64", (9, 1, 33), "wv", 0)
    assert a == b
    # unaligned columns fall back to scalar lanes
    assert xr.xr_plan_describe("+", "fp32", (100, 1, 33), "g", 256)["vec"] == 1
    assert xr.xr_plan_describe("+", "fp32", (100, 1, 32), "g", 4)["vec"] == 1
    assert xr.xr_plan_describe("+", "fp32", (100, 1, 32), "g", 256)["vec"] == 4


@pytest.mark.parametrize("case", [
    ("R", (2**30, 1, 1), "gwv"), ("KR", (8, 1, 2**27), "v"), ("RK", (2**26, 1, 16), "g"),
    ("RKR", (2**14, 4, 2**12), "gv"), ("KRK", (2, 2**24, 8), "w")])
def test_plan_fp32_chain_cap(xr, case):
    """fp32 '+' keeps every accumulator's sequential chain <= 4096 (C9)."""
    _, dims, lv = case
    p = xr.xr_plan_describe("+", "fp32", dims, lv, 256)
    if p["kernel"] == "rkr":
        per_acc = p["cdims"][0] * p["cdims"][2] / p["splits"] / (32 * p["vec"])  # per lane accumulator: k range x vectors per row
    elif p["kernel"] == "rows":
        per_acc = p["cdims"][1] / (32 * p["vec"])  # one row per warp-wide fold, VEC chains per lane
    elif p["kernel"] in ("seg", "stream"):
        c = p["cdims"]
        work = {"R": c[0], "KR": c[1], "RKR": c[0] * c[2]}[p["shape"]]
        per_acc = work / p["splits"] / (p["group"] * p["vec"] * 4)
    elif p["kernel"] == "colflat":  # 4 accumulators per thread, one vector per 4 KiB round
        R = p["cdims"][0] if p["shape"] == "RK" else p["cdims"][1]
        K = p["cdims"][1] if p["shape"] == "RK" else p["cdims"][2]
        per_acc = R * K * 4 / 4096 / p["splits"] / 4
    else:  # col: 8 warps x 4 rows in flight; coltma: 4 row phases x 2 accumulators
        R = p["cdims"][0] if p["shape"] == "RK" else p["cdims"][1]
        per_acc = R / p["splits"] / (8 * 4 if p["kernel"] == "col" else 8)
    assert per_acc <= 4096 + 1


def test_plan_parallelism_and_workspace(xr):
    # big single outputs split across many CTAs, each with a ticketed partial
    p = xr.xr_plan_describe("+", "fp32", (2**30, 1, 1), "gwv", 256)
    assert p["splits"] >= 148 and p["tickets"] == 1 and p["ws_bytes"] == 4 * p["splits"]
    # many rows: no gang-tier combine needed
    q = xr.xr_plan_describe("+", "fp32", (32768, 1, 32768), "v", 256)
    assert q["splits"] == 1 and q["ws_bytes"] == 0
    # few long rows get split, but only with warp- or CTA-wide groups
    r = xr.xr_plan_describe("+", "fp32", (512, 1, 262144), "v", 256)
    assert r["splits"] > 1 and r["group"] >= 32
    for dims, lv in [((2**20, 4, 8), "gv"), ((3, 2**20, 5), "w")]:
        s = xr.xr_plan_describe("+", "fp32", dims, lv, 256)
        assert s["splits"] == 1 or s["group"] >= 32


# ------------------------------------------------------------------ shard plan (8e)
@pytest.mark.parametrize("op,coll,nccl", [("+", 1, 0), ("*", 1, 1), ("max", 1, 2), ("min", 1, 3),
                                          ("&&", 1, 3), ("||", 1, 2), ("&", 2, -1), ("|", 2, -1),
                                          ("^", 2, -1)])
def test_shard_plan_collectives(xr, op, coll, nccl):
    for lv in ["g", "gw", "gv", "gwv"]:
        i = xr.xr_shard_plan(op, "int64", (64, 8, 16), lv, 4, 2)
        assert (i["collective"], i["nccl_op"]) == (coll, nccl)
        assert i["global_count"] == i["local_count"] and i["out_offset"] == 0
        assert i["gang_offset"] == 128
    for lv in ["w", "v", "wv"]:
        i = xr.xr_shard_plan(op, "int64", (64, 8, 16), lv, 4, 3)
        assert i["collective"] == xr.COLL_ALLGATHER
        assert i["global_count"] == 4 * i["local_count"]
        assert i["out_offset"] == 3 * i["local_count"]


def test_shard_plan_init_merged_once(xr):
    m = xr.GANG | xr.INIT_FROM_OUT
    merges = [xr.xr_shard_plan("+", "fp32", (8, 2, 2), m, 8, r)["merge_init"] for r in range(8)]
    assert merges == [1] + [0] * 7
    m2 = xr.VECTOR | xr.INIT_FROM_OUT
    assert all(xr.xr_shard_plan("+", "fp32", (8, 2, 2), m2, 8, r)["merge_init"] for r in range(8))
    assert xr.xr_shard_plan("+", "fp32", (8, 2, 2), "g", 2, 0)["merge_init"] == 0
    with pytest.raises(xr.XReduceError):
        xr.xr_shard_plan("+", "fp32", (8, 2, 2), "g", 2, 2)


def test_plan_column_box_group_rules(xr):
    """Column TMA plans (DESIGN 6.0, r02 A/B): 8-byte split tiles take 256-B
    boxes (16 tiles of 32 columns for 512 kept fp64 columns), 4-byte ones
    1 KiB boxes (2 tiles of 256 fp32 columns); one gang-tier level while
    S <= 64 (tickets = tiles * 2), groups of 16 beyond (S = 444: 28 groups)."""
    p = xr.xr_plan_describe("*", "fp64", (512, 512, 512), "gw", 256)
    assert p["kernel"] == "coltma" and p["splits"] == 55 and p["units"] == 16 * 55
    assert p["tickets"] == 16 * 2
    q = xr.xr_plan_describe("*", "int32", (512, 512, 512), "gw", 256)
    assert q["kernel"] == "coltma" and q["splits"] == 444 and q["units"] == 2 * 444
    assert q["tickets"] == 2 * (28 + 1)
    r = xr.xr_plan_describe("*", "fp64", (512, 512, 512), "g", 256)  # whole-tile units, 1 KiB boxes
    assert r["kernel"] == "coltma" and r["splits"] == 1 and r["units"] == 262144 // 128
