"""N2: several reduction variables with mixed dtypes in ONE launch
(xr_reduce_multi) -- each output must equal the oracle's single reduction of
its own input (the definition is per variable)."""
import numpy as np
import pytest

import oracle
from datagen import recipes
from gpu_util import check, torch_dt

pytestmark = pytest.mark.gpu
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "&": "band", "|": "bor",
        "^": "bxor", "&&": "land", "||": "lor"}
VARS = [("+", "int32"), ("+", "fp64"), ("max", "fp32"), ("^", "int64"), ("&&", "fp32"), ("*", "int32"),
        ("min", "int64"), ("+", "fp32")]


def run_multi(vars_, dims, levels, inputs, inits=None):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    n = xr.xr_out_count(dims, levels)
    xs = [torch.from_numpy(x).cuda() for x in inputs]
    outs = [torch.zeros(max(n, 1), dtype=torch_dt(dt), device="cuda") for _, dt in vars_]
    mask = xr.mask_of(levels)
    if inits is not None:
        for o, i in zip(outs, inits):
            o[:n].copy_(torch.from_numpy(i))
        mask |= xr.INIT_FROM_OUT
    n0 = xr.xr_launch_count()
    st = xr.xr_reduce_multi([(op, dt, x.data_ptr() if x.numel() else 0, o.data_ptr())
                             for (op, dt), x, o in zip(vars_, xs, outs)], dims, mask,
                            torch.cuda.current_stream().cuda_stream)
    assert st == 0, xr.xr_strerror(st)
    torch.cuda.synchronize()
    return [o[:n].cpu().numpy() for o in outs], xr.xr_launch_count() - n0


@pytest.mark.parametrize("dims,levels", [((64, 64, 128), "v"), ((64, 64, 128), "gwv"), ((9, 70, 130), "wv"),
                                         ((37, 41, 123), "gv"), ((1 << 20, 1, 1), "gwv"), ((5, 1, 7), "w"),
                                         ((3, 2, 100003), "v")])
def test_multi_matches_per_variable_oracle(dims, levels):
    mask = oracle.mask_of(levels)
    inputs = [recipes.make(KIND[op], dims, mask, dt, 40 + k) for k, (op, dt) in enumerate(VARS)]
    inits = [recipes.make("ints", (oracle.out_count(dims, levels), 1, 1), 1, dt, 50 + k)
             for k, (_, dt) in enumerate(VARS)]
    outs, launches = run_multi(VARS, dims, levels, inputs, inits)
    assert launches == 1
    for (op, dt), x, init, got in zip(VARS, inputs, inits, outs):
        check(op, dt, dims, levels, got, x, init=init)


def test_multi_edge_cases():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    # a reduced extent of 0 -> every output = its init
    v = [("+", "int32"), ("max", "fp64")]
    inits = [np.arange(12, dtype=np.int32), np.full(12, 2.5)]
    outs, _ = run_multi(v, (4, 0, 3), "w", [np.zeros(0, np.int32), np.zeros(0)], inits)
    assert outs[0].tolist() == inits[0].tolist() and outs[1].tolist() == inits[1].tolist()
    # column shapes are unsupported, bitwise on fp is unsupported, too many variables invalid
    t = torch.zeros(64, device="cuda")
    o = torch.zeros(64, device="cuda")
    assert xr.xr_reduce_multi([("+", "fp32", t.data_ptr(), o.data_ptr())], (4, 4, 4), "g") == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce_multi([("&", "fp32", t.data_ptr(), o.data_ptr())], (64, 1, 1), "g") == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce_multi([("+", "fp32", t.data_ptr(), o.data_ptr())] * 9, (64, 1, 1), "g") == xr.ERR_INVALID
    # an output overlapping another variable's input is rejected
    assert xr.xr_reduce_multi([("+", "fp32", t.data_ptr(), o.data_ptr()),
                               ("+", "fp32", o.data_ptr(), t.data_ptr() + 4)], (64, 1, 1), "g") == xr.ERR_INVALID
