"""GPU parity of the packed gang tier (xr_ops.cuh PackedAdd): 32-bit integer
'+' split across CTAs / warps keeps an output's running sum and arrival count
in ONE 64-bit word, so a split deposits its partial and takes its ticket with
a single atomic.  Checked bit-exact against the oracle (PAPER.md 3.1.3 @24887:
the gang partials' global combine; the result is the nest's sum mod 2^32, the
wrap the oracle computes), on values spanning the whole int32 range so every
sum wraps, on both seg group widths (warp, CTA), with the caller's init, on
back-to-back calls (the word self-resets) and against the ticket + partials
path (XR_NO_PACKED=1).
"""
import numpy as np
import pytest

import datagen
from gpu_util import check, gpu_reduce

pytestmark = pytest.mark.gpu

# (dims, mask, seg group width) -- plans checked below to be packed seg plans
CASES = [
    ((64, 64, 128), "gwv", 256),     # cfg1 testsuite nest: one unit per CTA
    ((64, 64, 128), "wv", 32),       # 32 KiB rows: warp groups, 16 splits per output
    ((64, 64, 128), "gv", 32),       # warp groups, 16 splits per output
    ((1, 1, 3000001), "gwv", 256),   # ragged whole array
    ((33, 1, 77777), "v", 256),      # long ragged rows split per CTA
    ((300, 41, 129), "gv", 32),      # RKR with odd rows
    ((7, 9000, 5), "wv", 256),
]


def _plan(xr, dims, lv):
    return xr.xr_plan_describe("+", "int32", dims, lv, 256)


@pytest.mark.parametrize("dims,lv,group", CASES)
def test_packed_int32_sum_wraps(dims, lv, group):
    import paper_conf_ppopp_xutycc14_b200 as xr
    p = _plan(xr, dims, lv)
    assert p["kernel"] == "seg" and p["splits"] > 1 and p["group"] == group, p
    assert p["tickets"] == 2 * p["out_count"] and p["ws_bytes"] == 0, p
    n = int(np.prod(dims))
    x = datagen.uniform_int(5151 + n % 97, n, -(1 << 31), (1 << 31) - 1, np.int32)
    got = gpu_reduce("+", "int32", dims, lv, x)
    check("+", "int32", dims, lv, got, x)
    # the word self-resets: a second call (and one merging init) are exact too
    again = gpu_reduce("+", "int32", dims, lv, x)
    assert np.array_equal(got, again)
    init = datagen.uniform_int(99, max(1, p["out_count"]), -(1 << 31), (1 << 31) - 1, np.int32)
    check("+", "int32", dims, lv, gpu_reduce("+", "int32", dims, lv, x, init=init), x, init=init)


@pytest.mark.parametrize("dims,lv,group", CASES[:3])
def test_packed_matches_ticket_path(monkeypatch, dims, lv, group):
    import paper_conf_ppopp_xutycc14_b200 as xr
    n = int(np.prod(dims))
    x = datagen.uniform_int(77, n, -(1 << 31), (1 << 31) - 1, np.int32)
    packed = gpu_reduce("+", "int32", dims, lv, x, offset=1)
    monkeypatch.setenv("XR_NO_PACKED", "1")
    q = _plan(xr, dims, lv)
    assert q["tickets"] == q["out_count"] and q["ws_bytes"] > 0, q
    ticket = gpu_reduce("+", "int32", dims, lv, x, offset=1)
    assert np.array_equal(packed, ticket)
    check("+", "int32", dims, lv, ticket, x)


def test_packed_graph_replay():
    """Captured once, replayed 50 times on changing inputs: every replay exact."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    dims, lv = (64, 64, 128), "gwv"
    n = int(np.prod(dims))
    xs = [datagen.uniform_int(300 + k, n, -(1 << 31), (1 << 31) - 1, np.int32) for k in range(5)]
    dev = torch.empty(n, dtype=torch.int32, device="cuda")
    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        dev.copy_(torch.from_numpy(xs[0]))
        assert xr.xr_reduce("+", "int32", dims, xr.mask_of(lv), dev.data_ptr(), out.data_ptr(), s.cuda_stream) == 0
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        assert xr.xr_reduce("+", "int32", dims, xr.mask_of(lv), dev.data_ptr(), out.data_ptr(), s.cuda_stream) == 0
    for k in range(50):
        x = xs[k % len(xs)]
        dev.copy_(torch.from_numpy(x))
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        check("+", "int32", dims, lv, out.cpu().numpy(), x)


# flat column kernel (RK / KRK with narrow rows): one packed word per output column
FLAT = [
    ((64, 64, 128), "gw"),           # cfg1 testsuite nest at gang + worker
    ((1 << 20, 2, 32), "g"),         # the paper's 2^20 x 2 x 32 gang case: 1184 splits per column
    ((3000, 1, 64), "g"),
    ((9, 4000, 32), "w"),            # KRK: 9 batches
    ((100000, 1, 4), "g"),           # 16-B rows
]


@pytest.mark.parametrize("dims,lv", FLAT)
def test_packed_colflat_int32_sum(dims, lv):
    import paper_conf_ppopp_xutycc14_b200 as xr
    p = _plan(xr, dims, lv)
    assert p["kernel"] == "colflat" and p["splits"] > 1, p
    assert p["tickets"] == 2 * p["out_count"] and p["ws_bytes"] == 0, p
    n = int(np.prod(dims))
    x = datagen.uniform_int(6161 + n % 89, n, -(1 << 31), (1 << 31) - 1, np.int32)
    got = gpu_reduce("+", "int32", dims, lv, x)
    check("+", "int32", dims, lv, got, x)
    assert np.array_equal(got, gpu_reduce("+", "int32", dims, lv, x))  # self-reset
    init = datagen.uniform_int(98, p["out_count"], -(1 << 31), (1 << 31) - 1, np.int32)
    check("+", "int32", dims, lv, gpu_reduce("+", "int32", dims, lv, x, init=init), x, init=init)
