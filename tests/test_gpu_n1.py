"""GPU parity for N1 (transform-reduce): Monte Carlo pi counts must equal the
oracle EXACTLY (both sides decide x*x + y*y < 1 in the inputs' precision, no
FMA); inner products within the C9 bound, ints exactly."""
import math

import numpy as np
import pytest

import datagen
import oracle
from gpu_util import TAU, torch_dt

pytestmark = pytest.mark.gpu
SEG_MASKS = ["v", "wv", "gv", "gwv"]   # canonical R / KR / RKR for 3 non-unit dims
COL_MASKS = ["g", "w", "gw"]           # canonical RK / KRK (column units, xr_colunit.cuh)
ALL_MASKS = SEG_MASKS + COL_MASKS


def run(xform, dtype, dims, levels, x, y, init=None, offset=0):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    bx = torch.empty(x.size + offset + 1, dtype=torch_dt(dtype), device="cuda")
    by = torch.empty(y.size + offset + 1, dtype=torch_dt(dtype), device="cuda")
    dx, dy = bx[offset:offset + x.size], by[offset:offset + y.size]
    dx.copy_(torch.from_numpy(x))
    dy.copy_(torch.from_numpy(y))
    n = xr.xr_out_count(dims, levels)
    odt = torch.int64 if xform == "disk" else torch_dt(dtype)
    out = torch.zeros(max(n, 1), dtype=odt, device="cuda")
    mask = xr.mask_of(levels)
    if init is not None:
        out[:n].copy_(torch.from_numpy(np.asarray(init)))
        mask |= xr.INIT_FROM_OUT
    st = xr.xr_transform_reduce(xform, dtype, dims, mask, dx.data_ptr(), dy.data_ptr(), out.data_ptr(),
                                torch.cuda.current_stream().cuda_stream)
    if st:
        raise xr.XReduceError(st, "xr_transform_reduce")
    torch.cuda.synchronize()
    return out[:n].cpu().numpy()


@pytest.mark.parametrize("dtype", ["fp32", "fp64"])
def test_disk_exact_counts_all_masks(dtype):
    # ragged column widths (129: scalar column lanes; 128: 16-B column lanes;
    # offset 1 misaligns both inputs), long reduced columns (5 x 70001 x 8)
    for dims in [(7, 33, 129), (3, 5, 100003), (64, 64, 128), (5, 70001, 8), (9000, 3, 36)]:
        n = int(np.prod(dims))
        x = datagen.uniform_float(1, n, -1.0, 1.0, oracle.NP_DTYPES[dtype])
        y = datagen.uniform_float(2, n, -1.0, 1.0, oracle.NP_DTYPES[dtype])
        for lv in ALL_MASKS:
            for off in (0, 1):
                init = np.arange(oracle.out_count(dims, lv), dtype=np.int64) * 3
                got = run("disk", dtype, dims, lv, x, y, init=init, offset=off)
                ref = oracle.transform_reduce("disk", dtype, dims, lv, x, y, init=init)
                assert np.array_equal(got, ref), (dims, lv, off)


def test_disk_lattice_and_boundary():
    N = 512
    i = np.arange(-N, N, dtype=np.int64)
    I, J = np.meshgrid(i, i, indexing="ij")
    x = (I / N).astype(np.float32).reshape(-1)
    y = (J / N).astype(np.float32).reshape(-1)
    got = run("disk", "fp32", (x.size, 1, 1), "g", x, y)
    assert got.tolist() == [int(np.count_nonzero(I * I + J * J < N * N))]
    b = np.array([0.6, 1.0, 0.0], np.float32)
    c = np.array([0.8, 0.0, 0.0], np.float32)
    assert run("disk", "fp32", (3, 1, 1), "g", b, c).tolist() == [1]   # on the circle: not counted


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
def test_dot_all_masks(dtype):
    dt = oracle.NP_DTYPES[dtype]
    for dims in [(9, 17, 300), (2, 3, 70001), (40, 33, 65), (3, 40000, 12)]:
        n = int(np.prod(dims))
        if dtype.startswith("int"):
            x = datagen.uniform_int(3, n, -1000, 1000, dt)
            y = datagen.uniform_int(4, n, -1000, 1000, dt)
        else:
            x = datagen.uniform_float(3, n, -1.0, 1.0, dt)
            y = datagen.uniform_float(4, n, -1.0, 1.0, dt)
        for lv in ALL_MASKS:
            for off in (0, 1):
                got = run("dot", dtype, dims, lv, x, y, offset=off)
                ref, S = oracle.transform_reduce("dot", dtype, dims, lv, x, y, want_abs=True)
                if dtype.startswith("int"):
                    assert np.array_equal(got, ref), (dims, lv, off)
                else:
                    err = np.abs(got.astype(np.float64) - ref.astype(np.float64))
                    assert np.all(err <= TAU[dtype] * S), (dims, lv, off)


def test_dot_column_init_and_empty():
    """Column shapes merge init once per output; an empty reduced extent gives out = init."""
    x = datagen.uniform_int(5, 6 * 50 * 40, -50, 50, np.int64)
    y = datagen.uniform_int(6, 6 * 50 * 40, -50, 50, np.int64)
    for lv in COL_MASKS:
        init = np.arange(oracle.out_count((6, 50, 40), lv), dtype=np.int64) - 7
        got = run("dot", "int64", (6, 50, 40), lv, x, y, init=init)
        assert np.array_equal(got, oracle.transform_reduce("dot", "int64", (6, 50, 40), lv, x, y, init=init))
    init = np.arange(6 * 40, dtype=np.int64)
    e = np.zeros(0, np.int64)
    assert np.array_equal(run("dot", "int64", (6, 0, 40), "w", e, e, init=init), init)


def test_unsupported_dtypes():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    out = torch.zeros(64, device="cuda")
    xi = torch.zeros(8, dtype=torch.int32, device="cuda")
    assert xr.xr_transform_reduce("disk", "int32", (8, 1, 1), "g", xi.data_ptr(), xi.data_ptr(),
                                  out.data_ptr()) == xr.ERR_UNSUPPORTED


@pytest.mark.slow
def test_monte_carlo_pi_4gb():
    """The paper's largest sample set: 4 GB of fp32 (x, y) pairs = 2^29 samples
    (reading C18); exact count vs the oracle, and pi within 5 sigma (P15)."""
    n = 1 << 29
    x = datagen.uniform_float(20140215, n, -1.0, 1.0, np.float32)
    y = datagen.uniform_float(20140216, n, -1.0, 1.0, np.float32)
    got = int(run("disk", "fp32", (n, 1, 1), "gv", x, y)[0])
    assert got == int(oracle.transform_reduce("disk", "fp32", (n, 1, 1), "gv", x, y)[0])
    p = math.pi / 4
    assert abs(4 * got / n - math.pi) <= 5 * 4 * math.sqrt(p * (1 - p) / n)
