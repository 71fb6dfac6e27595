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
                                         ((3, 2, 100003), "v"), ((64, 64, 128), "g"), ((64, 64, 128), "w"),
                                         ((9, 70, 130), "gw"), ((3, 20000, 36), "w"), ((30001, 2, 8), "g"),
                                         ((4096, 1, 20), "v"), ((1000, 3, 7), "v"), ((16, 1, 1000), "v"),
                                         ((7, 9, 1000), "gv")])
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
    # bitwise on fp is unsupported, too many variables invalid
    t = torch.zeros(64, device="cuda")
    o = torch.zeros(64, device="cuda")
    assert xr.xr_reduce_multi([("&", "fp32", t.data_ptr(), o.data_ptr())], (64, 1, 1), "g") == xr.ERR_UNSUPPORTED
    assert xr.xr_reduce_multi([("+", "fp32", t.data_ptr(), o.data_ptr())] * 9, (64, 1, 1), "g") == xr.ERR_INVALID
    # an output overlapping another variable's input is rejected
    assert xr.xr_reduce_multi([("+", "fp32", t.data_ptr(), o.data_ptr()),
                               ("+", "fp32", o.data_ptr(), t.data_ptr() + 4)], (64, 1, 1), "g") == xr.ERR_INVALID


def run_multi_at(vars_, dims, inputs, inits):
    """vars_: (op, dtype, levels); inits[k] None or the per-output init."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    xs = [torch.from_numpy(x).cuda() for x in inputs]
    outs, masks = [], []
    for (op, dt, lv), init in zip(vars_, inits):
        n = xr.xr_out_count(dims, lv)
        o = torch.zeros(max(n, 1), dtype=torch_dt(dt), device="cuda")
        m = xr.mask_of(lv)
        if init is not None:
            o[:n].copy_(torch.from_numpy(init))
            m |= xr.INIT_FROM_OUT
        outs.append((o, n))
        masks.append(m)
    n0 = xr.xr_launch_count()
    st = xr.xr_reduce_multi_at([(op, dt, m, x.data_ptr() if x.numel() else 0, o.data_ptr())
                                for (op, dt, _), m, x, (o, _) in zip(vars_, masks, xs, outs)], dims,
                               torch.cuda.current_stream().cuda_stream)
    assert st == 0, xr.xr_strerror(st)
    torch.cuda.synchronize()
    return [o[:n].cpu().numpy() for o, n in outs], xr.xr_launch_count() - n0


@pytest.mark.parametrize("dims", [(64, 64, 128), (9, 70, 130), (37, 41, 123), (3, 5000, 40), (1, 1, 100003)])
def test_multi_levels_per_variable(dims):
    """A7b (PAPER.md 3.2 @27198-27253): different variables reduced at different
    levels of one nest -- all 7 masks (row, column, batched-column, RKR and
    whole-nest shapes) with mixed ops / dtypes in ONE launch, each output equal
    to the oracle's reduction of its own input at its own levels."""
    LV = ["v", "w", "g", "wv", "gw", "gv", "gwv", "w"]
    mix = VARS
    vars_ = [(op, dt, lv) for (op, dt), lv in zip(mix, LV)]
    inputs = [recipes.make(KIND[op], dims, oracle.mask_of(lv), dt, 60 + k) for k, (op, dt, lv) in enumerate(vars_)]
    inits = [None if k % 2 else recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dt, 70 + k)
             for k, (_, dt, lv) in enumerate(vars_)]
    outs, launches = run_multi_at(vars_, dims, inputs, inits)
    assert launches == 1
    for (op, dt, lv), x, init, got in zip(vars_, inputs, inits, outs):
        check(op, dt, dims, lv, got, x, init=init)


def test_multi_levels_shared_input():
    """The paper's Fig 4 pattern on ONE array: per-row (vector), per-column
    (worker) and whole-nest sums of the same input in one launch."""
    dims = (16, 48, 96)
    x = recipes.make("ints", dims, 7, "int32", 80)
    vars_ = [("+", "int32", "v"), ("+", "int32", "w"), ("+", "int32", "gwv"), ("max", "int32", "gw")]
    outs, launches = run_multi_at(vars_, dims, [x] * 4, [None] * 4)
    assert launches == 1
    for (op, dt, lv), got in zip(vars_, outs):
        check(op, dt, dims, lv, got, x)


def test_multi_levels_edge_cases():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    # one variable with an empty output, one with a zero reduced extent, one identity
    dims = (4, 0, 3)
    z = np.zeros(0, np.int32)
    vars_ = [("+", "int32", "g"), ("+", "int32", "w"), ("max", "int32", "v")]
    init = np.arange(12, dtype=np.int32)
    outs, _ = run_multi_at(vars_, dims, [z, z, z], [None, init, None])
    assert outs[0].size == 0 and outs[1].tolist() == init.tolist() and outs[2].size == 0
    x = np.arange(4 * 3, dtype=np.int64).reshape(4, 1, 3).reshape(-1)
    outs, _ = run_multi_at([("+", "int64", "w"), ("*", "int64", "gv")], (4, 1, 3), [x, x + 1], [x.copy(), None])
    assert outs[0].tolist() == (2 * x).tolist()
    assert outs[1].tolist() == [int(np.prod(x + 1))]
    # a bad mask on any variable is invalid; fp bitwise unsupported
    t = torch.zeros(64, device="cuda")
    o = torch.zeros(64, device="cuda")
    assert xr.xr_reduce_multi_at([("+", "fp32", "gwv", t.data_ptr(), o.data_ptr()),
                                  ("+", "fp32", 0, t.data_ptr(), o.data_ptr() + 4)], (64, 1, 1)) == xr.ERR_INVALID
    assert xr.xr_reduce_multi_at([("|", "fp64", "g", t.data_ptr(), o.data_ptr())], (8, 1, 1)) == xr.ERR_UNSUPPORTED
    # two outputs overlapping
    assert xr.xr_reduce_multi_at([("+", "fp32", "v", t.data_ptr(), o.data_ptr()),
                                  ("+", "fp32", "v", t.data_ptr(), o.data_ptr() + 4)], (8, 1, 8)) == xr.ERR_INVALID
