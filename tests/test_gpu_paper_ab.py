"""N3: the paper-faithful kernels (xr_reduce_paper) must match the oracle like
xr_reduce does -- same output layout and init semantics (Table 2's positions,
ops and types), including ragged extents (NJ % num_workers != 0, the Fig 5a
barrier hazard) and non-default launch shapes."""
import numpy as np
import pytest

import oracle
from datagen import recipes
from gpu_util import check, torch_dt

pytestmark = pytest.mark.gpu


def run_paper(op, dtype, dims, levels, x, init=None, launch=(0, 0, 0)):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    xd = torch.from_numpy(x).cuda()
    n = xr.xr_out_count(dims, levels)
    out = torch.zeros(n, dtype=torch_dt(dtype), device="cuda")
    mask = xr.mask_of(levels)
    if init is not None:
        out.copy_(torch.from_numpy(init))
        mask |= xr.INIT_FROM_OUT
    st = xr.xr_reduce_paper(op, dtype, dims, mask, xd.data_ptr(), out.data_ptr(), *launch,
                            stream=torch.cuda.current_stream().cuda_stream)
    assert st == 0, xr.xr_strerror(st)
    torch.cuda.synchronize()
    return out.cpu().numpy()


@pytest.mark.parametrize("dtype", ["int32", "fp32", "fp64"])
@pytest.mark.parametrize("op", ["+", "*", "max"])
def test_paper_kernels_match_oracle(op, dtype):
    kind = {"+": "ints", "*": "mul", "max": "maxmin"}[op]
    for dims in [(64, 64, 128), (5, 13, 1000), (300, 2, 32), (3, 37, 77)]:
        for lv in ["g", "w", "v", "gw", "wv", "gwv"]:
            x = recipes.make(kind, dims, oracle.mask_of(lv), dtype, 7)
            init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 8)
            check(op, dtype, dims, lv, run_paper(op, dtype, dims, lv, x, init=init), x, init=init)


def test_paper_kernels_launch_shapes_and_errors():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    dims = (33, 19, 250)
    x = recipes.make("ints", dims, 7, "int32", 3)
    for launch in [(192, 8, 128), (148 * 16, 4, 256), (7, 1, 32), (1, 32, 32)]:
        for lv in ["g", "w", "v", "gw", "wv", "gwv"]:
            check("+", "int32", dims, lv, run_paper("+", "int32", dims, lv, x, launch=launch), x)
    t = torch.zeros(8, device="cuda")
    assert xr.xr_reduce_paper("&", "int32", (2, 2, 2), "g", t.data_ptr(), t.data_ptr()) == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce_paper("+", "fp32", (2, 2, 2), "gv", t.data_ptr(), t.data_ptr()) == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce_paper("+", "fp32", (2, 2, 2), "g", t.data_ptr(), t.data_ptr(), 4, 3, 100) == \
        xr.ERR_INVALID
