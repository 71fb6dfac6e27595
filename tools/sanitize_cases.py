#!/usr/bin/env python3
"""Small invocations of every kernel family, for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck).  Exits non-zero on a parity error."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402  (test infrastructure: checks the results)
import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402
from datagen import recipes  # noqa: E402
from gpu_util import check, gpu_reduce  # noqa: E402

cases = [
    ("+", "fp32", (1 << 18, 1, 1), "gwv"),        # stream (R)
    ("max", "int32", (64, 1, 1 << 14), "v"),      # stream (KR, 64 KiB rows)
    ("+", "fp32", (300, 1, 512), "v"),            # rows kernel
    ("^", "int64", (37, 41, 123), "v"),           # seg W=32
    ("*", "int32", (5, 3, 31), "v"),              # seg W=8
    ("+", "fp64", (40, 33, 700), "gv"),           # seg RKR split
    ("&&", "fp32", (700, 1, 512), "g"),           # coltma
    ("min", "fp32", (999, 1, 33), "g"),           # col (unaligned)
    ("|", "int32", (20, 300, 64), "w"),           # col KRK
    ("+", "int32", (3, 1, 5), "w"),               # ident
    ("+", "int32", (64, 64, 128), "g"),           # colsmall (r02)
    ("max", "fp64", (40, 33, 100), "w"),          # colsmall KRK, half-width last group
]
# r02: packed (sum, count) gang tier of the seg and flat column kernels
cases += [
    ("+", "int32", (64, 64, 128), "gwv"),         # seg W=CTA, packed, one unit per CTA
    ("+", "int32", (64, 64, 128), "gv"),          # seg W=32, packed
    ("+", "int32", (3000, 1, 64), "g"),           # colflat, packed
]
# staged kernels on small inputs (XR_SMALL_BYTES=0): column TMA kernel with
# 256-B boxes + split-major units (8-byte split tiles), 1 KiB boxes, rkr
staged = [
    ("*", "fp64", (4096, 1, 512), "g"),           # coltma, 256-B boxes, S > 1, split-major
    ("&&", "fp32", (700, 1, 512), "g"),           # coltma, 1 KiB boxes, S > 1
    ("^", "int64", (2000, 3, 512), "w"),          # coltma KRK, S == 1
    ("max", "int32", (40, 64, 256), "gv"),        # rkr
]
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "^": "bxor", "&&": "land", "|": "bor"}
for op, dtype, dims, lv in cases:
    x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, 1)
    check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x), x)
os.environ["XR_SMALL_BYTES"] = "0"
for op, dtype, dims, lv in staged:
    x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, 1)
    check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x), x)
del os.environ["XR_SMALL_BYTES"]
# heat (bulk + register variants), transform-reduce, multi, paper kernels
for nj, ni in [(70, 1030), (33, 67), (9, 5), (41, 1027)]:  # odd ni: shifted bulk staging (clip at the buffer end)
    T0 = oracle.heat_init(nj, ni)
    t1 = torch.from_numpy(T0).cuda()
    t2 = t1.clone()
    res = torch.zeros(3, dtype=torch.float64, device="cuda")
    assert xr.xr_heat_run(nj, ni, 3, t1.data_ptr(), t2.data_ptr(), res.data_ptr()) == 0
    torch.cuda.synchronize()
    assert res.cpu().tolist() == oracle.heat(nj, ni, 3, T0)[1].tolist()
xs = torch.rand(1 << 16, device="cuda") * 2 - 1
ys = torch.rand(1 << 16, device="cuda") * 2 - 1
cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
assert xr.xr_transform_reduce("disk", "fp32", (1 << 16, 1, 1), "gwv", xs.data_ptr(), ys.data_ptr(), cnt.data_ptr()) == 0
torch.cuda.synchronize()
assert int(cnt.item()) == int(oracle.transform_reduce("disk", "fp32", (1 << 16, 1, 1), "gwv",
                                                      xs.cpu().numpy(), ys.cpu().numpy())[0])
o1 = torch.zeros(64, device="cuda")
o2 = torch.zeros(64, dtype=torch.int32, device="cuda")
xi = torch.arange(64 * 1000, dtype=torch.int32, device="cuda")
assert xr.xr_reduce_multi([("+", "fp32", xs.data_ptr(), o1.data_ptr()), ("max", "int32", xi.data_ptr(), o2.data_ptr())],
                          (64, 1, 1000), "v") == 0
pz = torch.zeros(64 * 32, device="cuda")
assert xr.xr_reduce_paper("+", "fp32", (8, 8, 1000), "w", xs.data_ptr(), pz.data_ptr(), 16, 8, 128) == 0
assert xr.xr_reduce_paper("+", "fp32", (8, 8, 1000), "gwv", xs.data_ptr(), pz.data_ptr(), 16, 8, 128) == 0
torch.cuda.synchronize()
# round 2: the cluster kernel (opt-in), the two-input and multi-variable rings
os.environ["XR_CLUSTER"] = "1"
x = recipes.make("ints", (1 << 17, 1, 1), 7, "int32", 3)
check("+", "int32", (1 << 17, 1, 1), "gwv", gpu_reduce("+", "int32", (1 << 17, 1, 1), "gwv", x), x)
del os.environ["XR_CLUSTER"]
n = 1 << 22  # 16 MiB per fp32 input: xform_stream_kernel
bx = torch.rand(n, device="cuda") * 2 - 1
by = torch.rand(n, device="cuda") * 2 - 1
assert xr.xr_transform_reduce("disk", "fp32", (n, 1, 1), "gwv", bx.data_ptr(), by.data_ptr(), cnt.data_ptr()) == 0
torch.cuda.synchronize()
assert int(cnt.item()) == int(oracle.transform_reduce("disk", "fp32", (n, 1, 1), "gwv", bx.cpu().numpy(),
                                                      by.cpu().numpy())[0])
mo = [torch.zeros(1, device="cuda") for _ in range(2)] + [torch.zeros(1, dtype=torch.int64, device="cuda")]
mi = torch.arange(n, dtype=torch.int64, device="cuda")
assert xr.xr_reduce_multi([("+", "fp32", bx.data_ptr(), mo[0].data_ptr()), ("max", "fp32", by.data_ptr(), mo[1].data_ptr()),
                           ("+", "int64", mi.data_ptr(), mo[2].data_ptr())], (n, 1, 1), "gwv") == 0  # multi_stream_kernel
torch.cuda.synchronize()
assert int(mo[2].item()) == n * (n - 1) // 2
print("sanitize cases OK")
