"""CUDA-graph capture of the hot path (launch-bound inner loops, e.g. the
cfg1 testsuite nest or the heat iteration): after xr_reserve / one warm-up
call, xr_reduce and xr_heat_step enqueue no allocation and no host sync, so
they can be captured and replayed; replays must stay correct (tickets and
scheduler counters self-reset)."""
import numpy as np
import pytest

import datagen
import oracle
from datagen import recipes

pytestmark = pytest.mark.gpu


def test_capture_and_replay_reductions():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    dims = (64, 64, 128)
    x = datagen.uniform_int(5, int(np.prod(dims)), -1000, 1000, np.int32)
    xd = torch.from_numpy(x).cuda()
    s = torch.cuda.Stream()
    outs = {lv: torch.zeros(xr.xr_out_count(dims, lv), dtype=torch.int32, device="cuda")
            for lv in ["g", "w", "v", "gwv"]}
    big = torch.rand(1 << 24, device="cuda")
    big_out = torch.zeros(1, device="cuda")
    with torch.cuda.stream(s):
        for lv, o in outs.items():
            assert xr.xr_reserve("+", "int32", dims, lv, s.cuda_stream) == 0
            assert xr.xr_reduce("+", "int32", dims, lv, xd.data_ptr(), o.data_ptr(), s.cuda_stream) == 0
        assert xr.xr_reduce("+", "fp32", (1 << 24, 1, 1), "gwv", big.data_ptr(), big_out.data_ptr(), s.cuda_stream) == 0
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for lv, o in outs.items():
            assert xr.xr_reduce("+", "int32", dims, lv, xd.data_ptr(), o.data_ptr(), s.cuda_stream) == 0
        assert xr.xr_reduce("+", "fp32", (1 << 24, 1, 1), "gwv", big.data_ptr(), big_out.data_ptr(), s.cuda_stream) == 0
    ref_big = None
    for rep in range(20):
        for o in outs.values():
            o.zero_()
        g.replay()
        torch.cuda.synchronize()
        for lv, o in outs.items():
            assert np.array_equal(o.cpu().numpy(), oracle.reduce("+", "int32", dims, lv, x)), (rep, lv)
        if ref_big is None:
            ref_big = big_out.item()
        assert big_out.item() == ref_big  # deterministic across replays


def test_capture_heat_iterations():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    nj, ni, iters = 130, 258, 10
    T0 = oracle.heat_init(nj, ni)
    _, ref_res = oracle.heat(nj, ni, iters, T0)
    t1 = torch.from_numpy(T0).cuda()
    t2 = t1.clone()
    res = torch.zeros(iters, dtype=torch.float64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):  # warm-up grows the workspace
        assert xr.xr_heat_step(nj, ni, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), s.cuda_stream) == 0
    torch.cuda.synchronize()
    t1.copy_(torch.from_numpy(T0))
    t2.copy_(torch.from_numpy(T0))
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        assert xr.xr_heat_run(nj, ni, iters, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), s.cuda_stream) == 0
    g.replay()
    torch.cuda.synchronize()
    assert res.cpu().tolist() == ref_res.tolist()
