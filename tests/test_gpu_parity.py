"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by
element, on seeded inputs shaped like the paper's workloads (DESIGN.md
"Input recipe").  Sizes span several tiles and ragged tails; full BASELINE
sizes are in test_gpu_fullsize.py."""
import itertools
import random

import numpy as np
import pytest

import datagen
from datagen import recipes
import oracle
from gpu_util import seg_len, check, gpu_reduce

pytestmark = pytest.mark.gpu

ALL_MASKS = ["g", "w", "v", "gw", "gv", "wv", "gwv"]
PAIRS = [(op, dt) for dt in ["int32", "int64", "fp32", "fp64"]
         for op in ["+", "*", "max", "min", "&&", "||"] + (["&", "|", "^"] if dt.startswith("int") else [])]
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "&": "band", "|": "bor",
        "^": "bxor", "&&": "land", "||": "lor"}


@pytest.fixture(params=["planned", "staged"])
def staging(request, monkeypatch):
    """Run a test twice: with the planner's small-input threshold (small nests
    use the register kernels) and with XR_SMALL_BYTES=0, which routes the same
    small, ragged, misaligned cases through the bulk/TMA staged kernels."""
    if request.param == "staged":
        monkeypatch.setenv("XR_SMALL_BYTES", "0")
    return request.param


@pytest.fixture(scope="module", autouse=True)
def lib():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ppopp_xutycc14_b200 as xr
    return xr


# ---------------------------------------------------------------- config 1
@pytest.mark.parametrize("levels", ["g", "w", "v", "gwv"])
@pytest.mark.parametrize("variant", ["ints", "linear", "ones"])
def test_cfg1_testsuite_nest(levels, variant):
    dims = (64, 64, 128)
    seed = datagen.case_seed(1, 0, 0, oracle.mask_of(levels), 1)
    x = recipes.make(variant, dims, oracle.mask_of(levels), "int32", seed)
    g = gpu_reduce("+", "int32", dims, levels, x)
    check("+", "int32", dims, levels, g, x)
    if variant == "linear" and levels == "gwv":
        assert g.tolist() == [-262144]  # P1


def test_cfg1_paper_literal_fig4():
    """Fig 4 (a)/(b)/(c) with XR_INIT_FROM_OUT (P16)."""
    NK, NJ, NI = 64, 64, 128
    x = datagen.uniform_int(16, NK * NJ * NI, -1000, 1000, np.int32)
    init_a = np.tile(np.arange(NJ, dtype=np.int32), NK)                       # i_sum = j
    check("+", "int32", (NK, NJ, NI), "v", gpu_reduce("+", "int32", (NK, NJ, NI), "v", x, init_a), x, init_a)
    init_b = np.repeat(np.arange(NK, dtype=np.int32), NI)                     # j_sum = k
    check("+", "int32", (NK, NJ, NI), "w", gpu_reduce("+", "int32", (NK, NJ, NI), "w", x, init_b), x, init_b)
    g = gpu_reduce("+", "int32", (NK, NJ, NI), "g", x)
    assert g.reshape(NJ, NI)[0, 0] == int(x.reshape(NK, NJ, NI)[:, 0, 0].astype(np.int64).sum())


# ---------------------------------------------------------------- op x dtype x mask
@pytest.mark.parametrize("op,dtype", PAIRS)
@pytest.mark.parametrize("dims", [(37, 41, 123), (3, 129, 1000), (130, 7, 33)])
def test_all_pairs_all_masks(op, dtype, dims, staging):
    for levels in ALL_MASKS:
        mask = oracle.mask_of(levels)
        seed = datagen.case_seed(5, oracle.OPS[op], oracle.DTYPES[dtype], mask, sum(dims))
        x = recipes.make(KIND[op], dims, mask, dtype, seed)
        g = gpu_reduce(op, dtype, dims, levels, x)
        check(op, dtype, dims, levels, g, x)


@pytest.mark.parametrize("dtype", ["fp32", "fp64"])
def test_fp_sums_exact_regime(dtype):
    """Integer-valued data: any order is exact, so the GPU must be bit-exact (P8)."""
    for dims in [(64, 64, 128), (5, 300, 701), (1000, 3, 17)]:
        for levels in ALL_MASKS:
            x = recipes.make("intvals", dims, 7, dtype, 88)
            check("+", dtype, dims, levels, gpu_reduce("+", dtype, dims, levels, x), x, exact=True)


@pytest.mark.parametrize("dtype", ["fp32", "fp64"])
@pytest.mark.parametrize("kind", ["u01", "um11", "mulgen"])
def test_fp_general_data(dtype, kind):
    """General (non-exact) fp data under the C9 / C10 bounds.  Reading C10
    defines the general-regime product bound on segments of at most 512
    factors (1 +- 1e-3), so '*' runs only the masks whose segment is <= 512;
    the (8, 8, 8) and (7, 9, 8) nests give every mask such a segment.  Longer
    product segments are covered by the exact regime (bit-exact)."""
    op = "*" if kind == "mulgen" else "+"
    shapes = [(64, 64, 128), (17, 1000, 33)] + ([(8, 8, 8), (7, 9, 8)] if op == "*" else [])
    for dims in shapes:
        for levels in ALL_MASKS:
            if op == "*" and seg_len(dims, levels) > 512:
                continue
            x = recipes.make(kind, dims, 7, dtype, 123)
            check(op, dtype, dims, levels, gpu_reduce(op, dtype, dims, levels, x), x)


@pytest.mark.parametrize("dtype", ["fp32", "fp64"])
def test_fp_products_exact_regime(dtype):
    for dims in [(8, 64, 4096), (100, 300, 7)]:
        for levels in ALL_MASKS:
            x = recipes.make("mul", dims, oracle.mask_of(levels), dtype, 99)
            check("*", dtype, dims, levels, gpu_reduce("*", dtype, dims, levels, x), x, exact=True)


@pytest.mark.parametrize("dtype", ["fp32", "fp64"])
@pytest.mark.parametrize("op", ["max", "min", "&&", "||", "+", "*"])
def test_fp_special_values(op, dtype, staging):
    """NaN, +-inf, +-0 and subnormals (C7, C8): bit-exact for max/min/&&/||."""
    for dims in [(33, 17, 65), (2, 2, 3000)]:
        for levels in ALL_MASKS:
            # products: specials on exact +-1/2/0.5 data; long U[-1,1) chains would
            # underflow in dtype but not in the oracle's wider type (outside C10)
            kind = "mulspecials" if op == "*" else "specials"
            x = recipes.make(kind, dims, oracle.mask_of(levels), dtype, 7)
            check(op, dtype, dims, levels, gpu_reduce(op, dtype, dims, levels, x), x)
    z = np.array([-0.0, 0.0, -0.0], dtype=oracle.NP_DTYPES[dtype])
    if op in ("max", "min"):
        check(op, dtype, (3, 1, 1), "g", gpu_reduce(op, dtype, (3, 1, 1), "g", z), z)


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("op", ["&&", "||"])
def test_logical_truth_bit_patterns(op, dtype, staging):
    """C8 truth (x != 0) on the bit patterns the kernels' nonzero-accumulator
    folds must classify: sign-only words (INT_MIN, -0.0), 64-bit values whose
    low or high word alone is nonzero (2^32, 1, subnormals), NaN payloads.
    Inputs: all truthy (&& -> 1), all falsy (|| -> 0), and sparse mixes."""
    rng = np.random.default_rng(808)
    npdt = oracle.NP_DTYPES[dtype]
    if dtype == "int32":
        truthy = np.array([np.iinfo(np.int32).min, 1, -1, 1 << 16, (1 << 31) - 1], dtype=np.int64).astype(np.int32)
        falsy = np.zeros(1, np.int32)
    elif dtype == "int64":
        truthy = np.array([np.iinfo(np.int64).min, 1 << 32, -(1 << 32), 1, (1 << 63) - 1, 0x80000000], dtype=np.int64)
        falsy = np.zeros(1, np.int64)
    else:
        ut = np.uint32 if dtype == "fp32" else np.uint64
        sign = ut(1) << ut(31 if dtype == "fp32" else 63)
        pats = [1, sign | ut(1), (ut(0xFF) << ut(23)) | ut(1) if dtype == "fp32" else (ut(0x7FF) << ut(52)) | ut(1)]
        if dtype == "fp64":
            pats += [ut(1) << ut(32), sign | (ut(1) << ut(32))]  # high word only (low word zero)
        truthy = np.array(pats, dtype=ut).view(npdt)
        falsy = np.array([0, sign], dtype=ut).view(npdt)  # +0, -0
    for dims in [(5, 7, 300), (3, 130, 33)]:
        n = int(np.prod(dims))
        for kind in ("truthy", "falsy", "mix"):
            if kind == "truthy":
                x = rng.choice(truthy, n)
            elif kind == "falsy":
                x = rng.choice(falsy, n)
            else:
                x = rng.choice(truthy, n)
                x[rng.random(n) < 0.002] = falsy[-1]
                y = rng.choice(falsy, n)
                y[rng.random(n) < 0.002] = truthy[0]
                x = y if op == "||" else x  # sparse truthy in falsy for ||, the reverse for &&
            x = np.ascontiguousarray(x.astype(npdt, copy=False))
            for levels in ALL_MASKS:
                check(op, dtype, dims, levels, gpu_reduce(op, dtype, dims, levels, x), x)


# ---------------------------------------------------------------- fuzz: ragged, misaligned
def test_fuzz_shapes_and_misalignment(staging):
    rng = random.Random(2014)
    sizes = [1, 2, 3, 31, 32, 33, 127, 128, 129, 1000, 4097]
    for trial in range(120):
        dims = tuple(rng.choice(sizes) for _ in range(3))
        while np.prod(dims) > 3_000_000:
            dims = tuple(rng.choice(sizes) for _ in range(3))
        op, dtype = rng.choice(PAIRS)
        levels = rng.choice(ALL_MASKS)
        mask = oracle.mask_of(levels)
        x = recipes.make(KIND[op], dims, mask, dtype, trial)
        off = rng.randrange(0, 4)
        init = None
        if rng.random() < 0.4:
            init = recipes.make(KIND[op], (oracle.out_count(dims, levels), 1, 1), 1, dtype, trial + 7)
        g = gpu_reduce(op, dtype, dims, levels, x, init=init, offset=off)
        check(op, dtype, dims, levels, g, x, init=init)


@pytest.mark.parametrize("op,dtype", PAIRS)
def test_init_from_out_every_pair(op, dtype, staging):
    dims = (9, 70, 130)
    for levels in ALL_MASKS:
        mask = oracle.mask_of(levels)
        x = recipes.make(KIND[op], dims, mask, dtype, 5)
        init = recipes.make("ints" if op not in ("&", "|", "^") else KIND[op],
                            (oracle.out_count(dims, levels), 1, 1), 1, dtype, 6)
        check(op, dtype, dims, levels, gpu_reduce(op, dtype, dims, levels, x, init=init), x, init=init)


# ---------------------------------------------------------------- degenerate cases
def test_empty_and_degenerate():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    # reduced extent 0 -> out = init (C17); && normalises init to 0/1
    init = np.arange(12, dtype=np.int32) - 3
    for op in ["+", "*", "max", "min", "&&", "||", "^"]:
        g = gpu_reduce(op, "int32", (4, 0, 3), "w", np.zeros(0, np.int32), init=init)
        check(op, "int32", (4, 0, 3), "w", g, np.zeros(0, np.int32), init=init)
        g2 = gpu_reduce(op, "int32", (4, 0, 3), "w", np.zeros(0, np.int32))
        check(op, "int32", (4, 0, 3), "w", g2, np.zeros(0, np.int32))
    # kept extent 0 -> nothing (status OK)
    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    assert xr.xr_reduce("+", "int32", (0, 5, 5), "w", 0, out.data_ptr()) == 0
    # all extents 1 / every reduced extent 1 (ident)
    for dims, lv in [((1, 1, 1), "gwv"), ((5, 1, 7), "w"), ((1, 9, 11), "g")]:
        x = datagen.uniform_int(3, int(np.prod(dims)), -9, 9, np.int32)
        init = datagen.uniform_int(4, oracle.out_count(dims, lv), -9, 9, np.int32)
        check("+", "int32", dims, lv, gpu_reduce("+", "int32", dims, lv, x, init=init), x, init=init)
        check("&&", "int32", dims, lv, gpu_reduce("&&", "int32", dims, lv, x), x)
    # unsupported + invalid map to exceptions in the binding
    with pytest.raises(xr.XReduceError) as e:
        xr.reduce(torch.ones(8, device="cuda"), "&", "gwv")
    assert e.value.status == xr.ERR_UNSUPPORTED


def test_binding_reduce_shapes():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    t = torch.arange(2 * 3 * 4, dtype=torch.int64, device="cuda").reshape(2, 3, 4)
    assert xr.reduce(t, "+", "v").shape == (2, 3)
    assert xr.reduce(t, "+", "gw").cpu().tolist() == t.sum((0, 1)).cpu().tolist()
    assert xr.reduce(t, "max", "gwv").item() == 23
    assert xr.reduce(t, "+", "v", init=torch.ones(2, 3, dtype=torch.int64)).cpu().tolist() == \
        (t.sum(2) + 1).cpu().tolist()


def test_deterministic_and_streams():
    """Fixed grids -> bit-identical fp results run to run; two streams at once."""
    import torch
    x = recipes.make("u01", (1, 1, 1 << 24), 4, "fp32", 1)
    a = gpu_reduce("+", "fp32", (1, 1, 1 << 24), "gwv", x)
    b = gpu_reduce("+", "fp32", (1, 1, 1 << 24), "gwv", x)
    assert a.view(np.uint32)[0] == b.view(np.uint32)[0]
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    y = recipes.make("um11", (64, 512, 512), 7, "fp32", 2)
    r1 = gpu_reduce("+", "fp32", (64, 512, 512), "gw", y, stream=s1)
    r2 = gpu_reduce("max", "fp32", (64, 512, 512), "v", y, stream=s2)
    check("+", "fp32", (64, 512, 512), "gw", r1, y)
    check("max", "fp32", (64, 512, 512), "v", r2, y)


def test_host_buffer_path():
    import paper_conf_ppopp_xutycc14_b200 as xr
    for op, dtype, dims, lv in [("+", "fp64", (300, 40, 77), "wv"), ("^", "int64", (5, 6, 100001), "v"),
                                ("min", "fp32", (1 << 20, 1, 1), "gwv")]:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, 3)
        out = np.zeros(oracle.out_count(dims, lv), oracle.NP_DTYPES[dtype])
        assert xr.xr_reduce_host(op, dtype, dims, lv, x.ctypes.data, out.ctypes.data) == 0
        check(op, dtype, dims, lv, out, x)


def test_launch_count_single_pass():
    """Exactly one kernel launch per xr_reduce call (no second launch)."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    x = torch.rand(1 << 22, device="cuda")
    xr.reduce(x, "+", "gwv")
    torch.cuda.synchronize()
    n0 = xr.xr_launch_count()
    for lv in ["g", "w", "v", "gw", "gv", "wv", "gwv"]:
        xr.reduce(x, "+", lv, nest=(64, 256, 256))
    torch.cuda.synchronize()
    assert xr.xr_launch_count() - n0 == 7


# ---------------------------------------------------------------- heat (config 4)
@pytest.mark.parametrize("nj,ni", [(8, 8), (130, 258), (67, 131), (3, 40), (300, 64), (9, 5), (41, 1027), (20, 515), (7, 2049)])
def test_heat_bitwise(nj, ni):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    iters = 25
    T0 = oracle.heat_init(nj, ni)
    ref_T, ref_res = oracle.heat(nj, ni, iters, T0)
    t1 = torch.from_numpy(T0).cuda()
    t2 = t1.clone()
    res = torch.zeros(iters, dtype=torch.float64, device="cuda")
    assert xr.xr_heat_run(nj, ni, iters, t1.data_ptr(), t2.data_ptr(), res.data_ptr(),
                          torch.cuda.current_stream().cuda_stream) == 0
    torch.cuda.synchronize()
    final = (t1 if iters % 2 == 0 else t2).cpu().numpy()
    assert res.cpu().numpy().tolist() == ref_res.tolist()
    assert np.array_equal(final.view(np.uint64), ref_T.view(np.uint64))
    if nj >= 6 and ni >= 6:
        assert res.cpu().numpy()[:3].tolist() == [0.25, 0.125, 0.078125]


# ---------------------------------------------------------------- sharded (single-device sim)
@pytest.mark.parametrize("op,dtype", [("+", "int64"), ("^", "int32"), ("max", "fp32"), ("&&", "fp64"),
                                      ("*", "int32"), ("+", "fp32"), ("|", "int64")])
def test_sharded_sim_matches_unsharded(op, dtype):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    G = 4
    local = (16, 12, 100)
    gdims = (local[0] * G, local[1], local[2])
    for levels in ALL_MASKS:
        mask = oracle.mask_of(levels)
        x = recipes.make(KIND[op], gdims, mask, dtype, 42)
        xs = torch.from_numpy(x).cuda()
        n_loc = int(np.prod(local))
        shards = [xs[r * n_loc:(r + 1) * n_loc] for r in range(G)]
        info = xr.xr_shard_plan(op, dtype, local, mask, G, 0)
        for with_init in (False, True):
            m = mask
            init = None
            out = torch.zeros(info["global_count"], dtype=xs.dtype, device="cuda")
            if with_init:
                init = recipes.make("ints", (info["global_count"], 1, 1), 1, dtype, 9)
                out.copy_(torch.from_numpy(init))
                m |= xr.INIT_FROM_OUT
            st = xr.xr_reduce_sharded_sim(op, dtype, local, m, [s.data_ptr() for s in shards],
                                          out.data_ptr(), torch.cuda.current_stream().cuda_stream)
            assert st == 0
            torch.cuda.synchronize()
            check(op, dtype, gdims, levels, out.cpu().numpy(), x, init=init)


@pytest.mark.parametrize("G,n_local,ni", [(4, 33, 130), (2, 64, 1024), (3, 20, 67), (8, 9, 520)])
def test_heat_sharded_sim_bitwise(G, n_local, ni):
    """Gang-row sharded heat (halo exchange + max combine) == the whole grid, bitwise."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    nj, iters = G * n_local, 12
    T0 = oracle.heat_init(nj, ni)
    ref_T, ref_res = oracle.heat(nj, ni, iters, T0)
    full = T0.reshape(nj, ni)
    t1s, t2s = [], []
    for r in range(G):
        slab = np.zeros((n_local + 2, ni))
        lo, hi = r * n_local - 1, (r + 1) * n_local + 1  # global rows of the slab incl. halos
        src_lo, src_hi = max(lo, 0), min(hi, nj)
        slab[src_lo - lo:src_hi - lo] = full[src_lo:src_hi]
        t1s.append(torch.from_numpy(slab.reshape(-1)).cuda())
        t2s.append(t1s[-1].clone())
    res = torch.zeros(iters, dtype=torch.float64, device="cuda")
    st = xr.xr_heat_run_sharded_sim(n_local, ni, iters, [t.data_ptr() for t in t1s],
                                    [t.data_ptr() for t in t2s], res.data_ptr(),
                                    torch.cuda.current_stream().cuda_stream)
    assert st == 0
    torch.cuda.synchronize()
    assert res.cpu().tolist() == ref_res.tolist()
    fin = t1s if iters % 2 == 0 else t2s
    got = np.concatenate([f.cpu().numpy().reshape(n_local + 2, ni)[1:n_local + 1] for f in fin])
    assert np.array_equal(got.view(np.uint64), ref_T.reshape(nj, ni).view(np.uint64))


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("row_bytes", [512, 1024, 2048, 4096, 8192, 16384])
def test_rows_kernel_short_rows(dtype, row_bytes, staging):
    """KR with power-of-two rows of 512 B .. 16 KiB (the bulk-streamed rows
    kernel), ragged row counts (not a multiple of rows per stage), with init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    L = row_bytes // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    for O, op in [(7, "+"), (1003, "max"), (4096 + 5, "&&")]:
        dims = (O, 1, L)
        plan = xr.xr_plan_describe(op, dtype, dims, "v", 256)
        x = recipes.make(KIND[op], dims, 4, dtype, O)
        init = recipes.make("ints", (O, 1, 1), 1, dtype, 2)
        check(op, dtype, dims, "v", gpu_reduce(op, dtype, dims, "v", x, init=init), x, init=init)
        if O >= 1003 and row_bytes <= 2048 and staging == "staged":
            assert plan["kernel"] == "rows"


def test_ring_kernels_stress_repeatable():
    """The bulk/TMA ring kernels (stream, rows, coltma, heat) reuse shared-memory
    stages released through mbarriers; a real write-after-read race would
    corrupt results nondeterministically.  Integer results must be identical to
    the oracle on every one of many back-to-back runs (compute-sanitizer
    racecheck cannot model mbarrier/async-proxy ordering, profiles/)."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    cases = [("+", "int32", (1 << 22, 1, 1), "gwv"), ("^", "int64", (64, 1, 1 << 15), "v"),
             ("+", "int32", (8192, 1, 512), "v"), ("|", "int32", (4096, 1, 2048), "g")]
    for op, dtype, dims, lv in cases:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, 77)
        ref = oracle.reduce(op, dtype, dims, lv, x)
        xd = torch.from_numpy(x).cuda()
        outs = [torch.empty(ref.size, dtype=xd.dtype, device="cuda") for _ in range(50)]
        for o in outs:  # back to back on one stream: stages are refilled under load
            assert xr.xr_reduce(op, dtype, dims, lv, xd.data_ptr(), o.data_ptr()) == 0
        torch.cuda.synchronize()
        for o in outs:
            assert np.array_equal(o.cpu().numpy(), ref), (op, dtype, dims, lv)


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("row_bytes", [16, 32, 128, 512, 2048, 4096])
def test_colflat_narrow_rows(dtype, row_bytes, staging):
    """RK / KRK with power-of-two narrow rows (the flat column kernel): every
    thread meets a fixed column group; ragged row counts; batches; init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    K = row_bytes // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    for dims, lv, op in [((5003, 1, K), "g", "+"), ((3, 1001, K), "w", "max"), ((70001, 1, K), "g", "^" if
                         dtype.startswith("int") else "*"), ((2, 40000, K), "w", "&&")]:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, sum(dims))
        init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 3)
        check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x, init=init), x, init=init)
        if row_bytes <= 512:
            assert xr.xr_plan_describe(op, dtype, dims, lv, 256)["kernel"] == "colflat"


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("row_bytes", [512, 1024, 2048])
@pytest.mark.parametrize("units", ["auto", "1", "64"])
def test_rkr_kernel_short_rows(dtype, row_bytes, units, monkeypatch):
    """RKR (gang + vector reduced, worker kept) with short rows: the rkr rows
    kernel (j-blocks of 16 KiB / row_bytes outputs streamed per k, per-warp
    register accumulation, per-output gang tier), forced with XR_SMALL_BYTES=0;
    ragged j-blocks (K not a multiple of the block), k split from 1 unit per
    CTA (few long units) to 64, with init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_SMALL_BYTES", "0")
    monkeypatch.setenv("XR_RKR_RING", "1")  # C >= O with 2 KiB rows would take the seg kernel
    if units != "auto":
        monkeypatch.setenv("XR_RKR_UNITS_PER_CTA", units)
    L = row_bytes // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    for R1, K, op in [(7, 32, "+"), (33, 100, "max"), (5, 999, "&&"), (300, 40, "*"), (64, 37, "||"),
                      (1, 64, "min")]:
        dims = (R1, K, L)
        x = recipes.make(KIND[op], dims, oracle.mask_of("gv"), dtype, R1 * K)
        init = recipes.make("ints", (K, 1, 1), 1, dtype, 4)
        check(op, dtype, dims, "gv", gpu_reduce(op, dtype, dims, "gv", x, init=init), x, init=init)
        if R1 > 1:
            assert xr.xr_plan_describe(op, dtype, dims, "gv", 256)["kernel"] == "rkr"
        if dtype.startswith("int"):
            xb = recipes.make("bxor", dims, oracle.mask_of("gv"), dtype, R1 + K)
            check("^", dtype, dims, "gv", gpu_reduce("^", dtype, dims, "gv", xb), xb)


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("row_bytes", [1024, 1536, 2048, 4096, 20480])
@pytest.mark.parametrize("splits", ["auto", "1", "3", "7"])
def test_stream_rkr_rows(dtype, row_bytes, splits, monkeypatch):
    """RKR (gang + vector reduced, worker kept) with 16-B aligned rows of >= 1 KiB:
    the stream kernel fills its stages from each unit's rows at the row stride
    (rows straddling stages when row_bytes does not divide 16 KiB, rows longer
    than a stage); ragged row splits (XR_STREAM_SPLITS), with init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_SMALL_BYTES", "0")
    monkeypatch.setenv("XR_RKR_STREAM_MIN_ROW", "1024")  # the planner's default is 4 KiB rows
    monkeypatch.setenv("XR_NO_RKR", "1")  # 1-2 KiB rows would take the rkr rows kernel
    monkeypatch.setenv("XR_RKR_RING", "1")  # C >= O with 2-4 KiB rows would take the seg kernel
    if splits != "auto":
        monkeypatch.setenv("XR_STREAM_SPLITS", splits)
    L = row_bytes // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    for R1, K, op in [(7, 3, "+"), (33, 100, "max"), (5, 129, "&&"), (61, 8, "*"), (19, 17, "||")]:
        dims = (R1, K, L)
        x = recipes.make(KIND[op], dims, oracle.mask_of("gv"), dtype, R1 * K + row_bytes)
        init = recipes.make("ints", (K, 1, 1), 1, dtype, 4)
        check(op, dtype, dims, "gv", gpu_reduce(op, dtype, dims, "gv", x, init=init), x, init=init)
        assert xr.xr_plan_describe(op, dtype, dims, "gv", 256)["kernel"] == "stream"
        if dtype.startswith("int"):  # & | ^ on the same path
            xb = recipes.make("bxor", dims, oracle.mask_of("gv"), dtype, R1 + K)
            check("^", dtype, dims, "gv", gpu_reduce("^", dtype, dims, "gv", xb), xb)


@pytest.mark.parametrize("box", ["256", "512", "1024"])
@pytest.mark.parametrize("order", ["split", "tile"])
@pytest.mark.parametrize("group", ["auto", "3"])
def test_coltma_box_order_group(box, order, group, monkeypatch):
    """The column TMA kernel's round-2 variants on ragged RK / KRK shapes, every
    dtype: TMA box width (256 / 512 / 1024 B x 16 KiB), split-major or
    tile-major unit ids, and the two-level gang tier with groups of 3 unit
    partials (many groups per tile, so the second level always runs), with
    init; each plan is checked to be the column TMA kernel with the forced
    settings."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_SMALL_BYTES", "0")
    monkeypatch.setenv("XR_COLTMA_BOX", box)
    if order == "tile":
        monkeypatch.setenv("XR_COLTMA_TILE_MAJOR", "1")
    if group != "auto":
        monkeypatch.setenv("XR_COLTMA_GROUP", group)
    cases = [("+", "fp32", (999, 1, 1000), "g"), ("max", "int32", (3, 301, 640), "w"),
             ("*", "fp64", (700, 1, 260), "g"), ("^", "int64", (2, 257, 1030), "w"),
             ("&&", "fp32", (4100, 1, 384), "g")]
    for op, dtype, dims, lv in cases:
        p = xr.xr_plan_describe(op, dtype, dims, lv, 256)
        assert p["kernel"] == "coltma", (dims, p)
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, sum(dims) + int(box))
        init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 5)
        check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x, init=init), x, init=init)


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("row_bytes", [16, 32, 64, 128, 256, 48, 80, 240, 496])
@pytest.mark.parametrize("units", ["auto", "1", "16"])
def test_rkr_narrow_rows(dtype, row_bytes, units, monkeypatch):
    """RKR with NARROW rows (16-496 B; powers of two and other multiples of
    16 B): the rkr kernel's narrow consumers (each thread meets the same 4
    rows of every stage of whole rows; rows combined by shuffles, or through
    shared memory when a row's vectors straddle warps; the row owners run the
    per-output gang tier), forced with
    XR_SMALL_BYTES=0; ragged j-blocks (outputs not a multiple of the J =
    16 KiB / row_bytes rows of a stage), k split from 1 unit per CTA to 16,
    with init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_SMALL_BYTES", "0")
    if units != "auto":
        monkeypatch.setenv("XR_RKR_UNITS_PER_CTA", units)
    L = row_bytes // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    J = 16384 // row_bytes
    for R1, K, op in [(7, J, "+"), (33, J + 5, "max"), (5, 2 * J + 1, "&&"), (64, J, "*"), (19, 3 * J - 7, "||"),
                      (1, J, "min")]:
        dims = (R1, K, L)
        x = recipes.make(KIND[op], dims, oracle.mask_of("gv"), dtype, R1 * K + row_bytes)
        init = recipes.make("ints", (K, 1, 1), 1, dtype, 4)
        check(op, dtype, dims, "gv", gpu_reduce(op, dtype, dims, "gv", x, init=init), x, init=init)
        if R1 > 1:
            assert xr.xr_plan_describe(op, dtype, dims, "gv", 256)["kernel"] == "rkr"
        if dtype.startswith("int"):
            xb = recipes.make("bxor", dims, oracle.mask_of("gv"), dtype, R1 + K)
            check("^", dtype, dims, "gv", gpu_reduce("^", dtype, dims, "gv", xb), xb)


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("row_bytes", [8, 16, 32, 64, 128])
def test_shortrow_kernel(dtype, row_bytes):
    """KR with short power-of-two rows (8-128 B): the short-row kernel (a thread
    per 64 / 128-B chunk of whole rows, rows folded in element order), every
    op, row counts that leave a partial last chunk, with init; a misaligned
    start takes the seg kernel instead (checked too)."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    size = np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    if row_bytes < 2 * size:
        pytest.skip("a row of one element is not a reduction")
    L = row_bytes // size
    for O, op in [(1, "+"), (7, "max"), (1000, "*"), (4099, "&&"), (65537, "||"), (333, "min")]:
        dims = (O, 1, L)
        x = recipes.make(KIND[op], dims, oracle.mask_of("v"), dtype, O + row_bytes)
        init = recipes.make("ints", (O, 1, 1), 1, dtype, 3)
        if O > 1:  # one row is the whole-array (R) shape
            assert xr.xr_plan_describe(op, dtype, dims, "v", 256)["kernel"] == "shortrow"
        check(op, dtype, dims, "v", gpu_reduce(op, dtype, dims, "v", x, init=init), x, init=init)
        check(op, dtype, dims, "v", gpu_reduce(op, dtype, dims, "v", x, offset=1), x)
        if dtype.startswith("int"):
            xb = recipes.make("bxor", dims, oracle.mask_of("v"), dtype, O)
            check("^", dtype, dims, "v", gpu_reduce("^", dtype, dims, "v", xb), xb)


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
@pytest.mark.parametrize("R", [2, 3, 5, 16, 32])
def test_thincol_kernel(dtype, R):
    """RK / KRK with few reduced rows (R <= 32) and >= 65536 kept 16-B column
    groups: the thin column kernel (a thread per column group folding its R
    rows in order), every op, with init; RK and KRK (batches)."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    vec = 16 // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    for dims, lv, op in [((R, 1, 65536 * vec), "g", "+"), ((R, 1, 65536 * vec + vec), "g", "max"),
                         ((3, R, 32768 * vec), "w", "*"), ((R, 1, 70000 * vec), "g", "&&"), ((5, R, 16384 * vec), "w", "||")]:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, R + dims[2])
        init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 6)
        assert xr.xr_plan_describe(op, dtype, dims, lv, 256)["kernel"] == "thincol", (dims, lv)
        check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x, init=init), x, init=init)
        if dtype.startswith("int"):
            xb = recipes.make("bxor", dims, oracle.mask_of(lv), dtype, R)
            check("^", dtype, dims, lv, gpu_reduce("^", dtype, dims, lv, xb), xb)


@pytest.mark.parametrize("dtype", ["int32", "fp32"])
@pytest.mark.parametrize("staging", ["planned", "staged"])
def test_colflat_two_columns(dtype, staging, monkeypatch):
    """RK / KRK with 8-B rows (two 32-bit columns): the flat column kernel with
    two whole rows per 16-B vector (lane q is column q % 2), odd row counts
    (a last 8-B row folded by scalar loads), batches with an even row count,
    every op, with init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    if staging == "staged":
        monkeypatch.setenv("XR_SMALL_BYTES", "0")
    for dims, lv, op in [((1, 99999, 2), "w", "+"), ((1000001, 1, 2), "g", "max"), ((3, 4096, 2), "w", "*"),
                         ((7, 513, 2), "gw", "&&"), ((2, 1000, 2), "w", "||"), ((123457, 1, 2), "g", "min")]:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, sum(dims))
        init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 8)
        assert xr.xr_plan_describe(op, dtype, dims, lv, 256)["kernel"] == "colflat", (dims, lv)
        check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x, init=init), x, init=init)
        if dtype == "int32":
            xb = recipes.make("bxor", dims, oracle.mask_of(lv), dtype, dims[1])
            check("^", dtype, dims, lv, gpu_reduce("^", dtype, dims, lv, xb), xb)
