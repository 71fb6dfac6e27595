"""GPU tests of the round-2 boundary work, all through the C ABI against the
oracle:

- xr_reduce_host's chunked pipeline (include/xreduce.h): inputs many times
  larger than the staging chunk, every mask, with and without init, and
  concurrent calls on different streams (per-(device, stream) staging);
- the TMA encode-failure fallback (re-plan onto the register column kernel);
- the fused exchange's bounded wait: a rank that never arrives makes the
  others time out, leave out unchanged and report XR_ERR_NCCL;
- the Python binding's validation on device tensors.
"""
import threading

import numpy as np
import pytest

import datagen
import oracle
from datagen import recipes
from gpu_util import check, gpu_reduce, torch_dt

pytestmark = pytest.mark.gpu
MASKS = ["g", "w", "v", "gw", "gv", "wv", "gwv"]
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "&": "band", "|": "bor", "^": "bxor",
        "&&": "land", "||": "lor"}


def host_reduce(op, dtype, dims, levels, x, init=None, stream=None):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    xin = torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
    n = xr.xr_out_count(dims, levels)
    out = np.zeros(max(n, 1), dtype=oracle.NP_DTYPES[dtype])
    mask = xr.mask_of(levels)
    if init is not None:
        out[:n] = init
        mask |= xr.INIT_FROM_OUT
    s = stream.cuda_stream if stream is not None else torch.cuda.current_stream().cuda_stream
    st = xr.xr_reduce_host(op, dtype, dims, mask, xin.data_ptr() if x.size else 0, out.ctypes.data, s)
    assert st == 0, xr.xr_strerror(st)
    return out[:n]


@pytest.mark.parametrize("op,dtype", [("+", "int32"), ("+", "fp32"), ("*", "int64"), ("max", "fp64"),
                                      ("^", "int64"), ("&&", "fp32"), ("min", "int32"), ("||", "int64")])
@pytest.mark.parametrize("chunk", [64, 4096, 1 << 20])
def test_reduce_host_chunked_every_mask(monkeypatch, op, dtype, chunk):
    """Inputs 10-1000x the chunk: several chunks per output block on every
    mask, the first merging the caller's init, the others accumulating."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_HOST_CHUNK_BYTES", str(chunk))
    dims = (37, 19, 23)
    for lv in MASKS:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, 41)
        nchunks = len(xr.xr_host_chunks(dims, lv, dtype, chunk))
        assert nchunks >= (x.nbytes // chunk), (nchunks, x.nbytes, chunk)
        got = host_reduce(op, dtype, dims, lv, x)
        check(op, dtype, dims, lv, got, x)
        init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 9)
        got = host_reduce(op, dtype, dims, lv, x, init=init)
        check(op, dtype, dims, lv, got, x, init=init)


def test_reduce_host_large_default_chunks():
    """256 MiB fp32 (8 default 32 MiB chunks) and a 33 MiB odd-sized int64
    array whose last chunk is partial."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    n = 1 << 26
    x = datagen.uniform_float(77, n, 0.0, 1.0, np.float32)
    assert len(xr.xr_host_chunks((n, 1, 1), "gwv", "fp32", 32 << 20)) == 8
    check("+", "fp32", (n, 1, 1), "gwv", host_reduce("+", "fp32", (n, 1, 1), "gwv", x), x)
    n2 = (33 << 20) // 8 + 3
    y = datagen.uniform_int(78, n2, -(1 << 40), 1 << 40, np.int64)
    for lv, dims in (("gwv", (n2, 1, 1)), ("v", (n2 // 3 // 1, 1, 3))):
        yy = y[:dims[0] * dims[2]]
        check("+", "int64", dims, lv, host_reduce("+", "int64", dims, lv, yy), yy)


def test_reduce_host_concurrent_streams(monkeypatch):
    """Two host threads on two streams: per-(device, stream) staging keeps
    their chunks apart (one shared staging buffer raced)."""
    import torch
    monkeypatch.setenv("XR_HOST_CHUNK_BYTES", str(1 << 16))
    dims = (64, 33, 129)
    xs = [datagen.uniform_int(200 + t, int(np.prod(dims)), -1000, 1000, np.int32) for t in range(2)]
    refs = [oracle.reduce("+", "int32", dims, "gw", x) for x in xs]
    streams = [torch.cuda.Stream() for _ in range(2)]
    errors = []

    def worker(t):
        try:
            torch.cuda.set_device(0)
            for _ in range(10):
                got = host_reduce("+", "int32", dims, "gw", xs[t], stream=streams[t])
                if not np.array_equal(got, refs[t]):
                    errors.append(t)
        except Exception as e:  # noqa: BLE001
            errors.append(repr(e))

    th = [threading.Thread(target=worker, args=(t,)) for t in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errors, errors


def test_reduce_host_empty_reduced_extent():
    got = host_reduce("+", "int32", (0, 3, 4), "g", np.zeros(0, dtype=np.int32), init=np.arange(12, dtype=np.int32))
    assert np.array_equal(got, np.arange(12, dtype=np.int32))  # C17: out = init


def test_tma_encode_failure_falls_back(monkeypatch):
    """XR_TEST_TMAP_FAIL makes the tensor-map encode fail: the call re-plans
    onto the register column kernel (one launch) and stays correct."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    dims = (1, 4096, 4096)  # 64 MiB: above the column TMA kernel's 48 MiB threshold
    x = datagen.uniform_int(5, int(np.prod(dims)), -(1 << 20), 1 << 20, np.int32)
    xd = torch.from_numpy(x).cuda()
    assert xr.xr_plan_describe("+", "int32", dims, "w", xd.data_ptr())["kernel"] == "coltma"
    monkeypatch.setenv("XR_TEST_TMAP_FAIL", "1")
    n0 = xr.xr_launch_count()
    got = xr.reduce(xd, "+", "w", nest=dims)
    torch.cuda.synchronize()
    assert xr.xr_launch_count() - n0 == 1
    assert np.array_equal(got.cpu().numpy().reshape(-1), oracle.reduce("+", "int32", dims, "w", x))


@pytest.mark.parametrize("G,skip", [(2, 1), (4, 0), (3, 2)])
def test_fused_exchange_times_out_without_stale_write(monkeypatch, G, skip):
    """One simulated rank never launches: the others' bounded waits expire,
    they leave out unchanged (no stale combine) and the call reports
    XR_ERR_NCCL.  The sim's per-stream warm-up leaves every out
    at its local sum n_local except rank 0's, restored to the caller's -7; a
    stale combine of the mailboxes would write (G - 1) * n_local instead."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_TEST_SIM_SKIP_RANK", str(skip))
    monkeypatch.setenv("XR_EXCH_TIMEOUT_MS", "300")
    n_local = 1 << 20
    xd = torch.ones(n_local * G, dtype=torch.int64, device="cuda")
    outs = [torch.full((1,), -7, dtype=torch.int64, device="cuda") for _ in range(G)]
    st = xr.xr_reduce_fused_sim("+", "int64", (n_local, 1, 1), 7,
                                [xd[r * n_local:(r + 1) * n_local].data_ptr() for r in range(G)],
                                [o.data_ptr() for o in outs])
    assert st == xr.ERR_NCCL
    assert [int(o.item()) for o in outs] == [-7] + [n_local] * (G - 1)
    monkeypatch.delenv("XR_TEST_SIM_SKIP_RANK")
    st = xr.xr_reduce_fused_sim("+", "int64", (n_local, 1, 1), 7,
                                [xd[r * n_local:(r + 1) * n_local].data_ptr() for r in range(G)],
                                [o.data_ptr() for o in outs])
    assert st == 0 and [int(o.item()) for o in outs] == [n_local * G] * G


def test_python_binding_validates_device_calls():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    x = torch.arange(24, dtype=torch.int32, device="cuda")
    with pytest.raises(ValueError):
        xr.reduce(x, "+", "g", nest=(5, 5, 1))                     # 25 != 24 elements
    with pytest.raises(ValueError):
        xr.reduce(x, "+", "g", nest=(2, 3, 4), out=torch.zeros(12, dtype=torch.int64, device="cuda"))
    with pytest.raises(ValueError):
        xr.reduce(x, "+", "g", nest=(2, 3, 4), out=torch.zeros(12, dtype=torch.int32))  # host out
    got = xr.reduce(x.reshape(2, 3, 2, 2), "+", "g")              # 4-D: leading dims flattened -> (6, 2, 2)
    assert got.cpu().tolist() == [[sum(range(k, 24, 4)) for k in range(j * 2, j * 2 + 2)] for j in range(2)]


@pytest.mark.parametrize("op,dtype", [("+", "int32"), ("+", "fp32"), ("*", "int64"), ("max", "fp64"),
                                      ("^", "int32"), ("&&", "fp32"), ("min", "int64"), ("||", "int32")])
def test_colsmall_kernel(op, dtype):
    """Small column shapes with few reduced rows (the cfg1 testsuite nest at
    gang / worker level): one warp per 32 B of kept columns, rows strided by
    lane (ragged R), a half-width last group (K % (2 VEC) != 0), batches, init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    vec = 16 // np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    cases = [((64, 64, 128), "g"), ((64, 64, 128), "w"), ((3, 601 * vec, 1), "g"),
             ((256, 515 * vec, 1), "g"), ((40, 33, 24 * vec + vec), "w"), ((7, 2, 300 * vec), "w"),
             ((31, 1, 2048 * vec), "g"), ((2, 65, 1024 * vec), "w")]
    for dims, lv in cases:
        x = recipes.make(KIND[op], dims, oracle.mask_of(lv), dtype, sum(dims) + 1)
        plan = xr.xr_plan_describe(op, dtype, dims, lv, 256)
        assert plan["kernel"] == "colsmall", (dims, lv, plan)
        check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x), x)
        init = recipes.make("ints", (oracle.out_count(dims, lv), 1, 1), 1, dtype, 5)
        check(op, dtype, dims, lv, gpu_reduce(op, dtype, dims, lv, x, init=init), x, init=init)


@pytest.mark.parametrize("xform,dtype", [("disk", "fp32"), ("disk", "fp64"), ("dot", "int32"), ("dot", "int64"),
                                         ("dot", "fp32"), ("dot", "fp64")])
def test_transform_reduce_bulk_ring(xform, dtype):
    """Whole-array transform-reduce on >= 16 MiB inputs: the two-input bulk
    ring (xform_stream_kernel).  Disk counts and integer dots are bit-exact
    against the oracle, fp dots within C9; a ragged tail (n % VEC != 0), init,
    and a misaligned pair that falls back to the register path."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    npd = oracle.NP_DTYPES[dtype]
    n = (16 << 20) // np.dtype(npd).itemsize + 3
    if dtype.startswith("fp"):
        x = datagen.uniform_float(61, n + 1, -1.0, 1.0, npd)
        y = datagen.uniform_float(62, n + 1, -1.0, 1.0, npd)
    else:
        x = datagen.uniform_int(61, n + 1, -1000, 1000, npd)
        y = datagen.uniform_int(62, n + 1, -1000, 1000, npd)
    xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    odt = torch.int64 if xform == "disk" else torch_dt(dtype)
    for off in (0, 1):  # 16-B aligned (bulk ring) and misaligned (register path)
        for init in (None, 7):
            out = torch.full((1,), 0 if init is None else init, dtype=odt, device="cuda")
            mask = xr.mask_of("gwv") | (xr.INIT_FROM_OUT if init is not None else 0)
            assert xr.xr_transform_reduce(xform, dtype, (n, 1, 1), mask, xd[off:].data_ptr(), yd[off:].data_ptr(),
                                          out.data_ptr(), torch.cuda.current_stream().cuda_stream) == 0
            ini = None if init is None else np.array([init], dtype=np.int64 if xform == "disk" else npd)
            ref, S = oracle.transform_reduce(xform, dtype, (n, 1, 1), "gwv", x[off:off + n], y[off:off + n],
                                             init=ini, want_abs=True)
            got = out.cpu().numpy()
            if xform == "disk" or not dtype.startswith("fp"):
                assert np.array_equal(got, ref), (xform, dtype, off, init, got, ref)
            else:
                tau = 1e-5 if dtype == "fp32" else 1e-12
                assert abs(float(got[0]) - float(ref[0])) <= tau * S[0], (got, ref, S)


def test_multi_variable_bulk_ring():
    """Eight whole-array variables of mixed (op, dtype) on a large nest: the
    multi-variable bulk ring (one launch); every output against the oracle
    (integer / bitwise / logical / min / max bit-exact, fp + and * within
    C9 / C10), with init on half of them, a ragged length, and the same call
    with one misaligned input (the register path)."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    n = (1 << 22) + 5
    vars_ = [("+", "int32"), ("+", "fp64"), ("max", "fp32"), ("^", "int64"), ("&&", "fp32"), ("*", "int32"),
             ("min", "int64"), ("+", "fp32")]
    for off in (0, 1):
        xs, ds, outs, inits, spec = [], [], [], [], []
        for k, (op, dt) in enumerate(vars_):
            x = recipes.make(KIND[op], (n + 1, 1, 1), 7, dt, 300 + k)
            xd = torch.from_numpy(x).cuda()
            init = recipes.make("ints", (1, 1, 1), 1, dt, 9 + k) if k % 2 == 0 else None
            o = torch.zeros(1, dtype=torch_dt(dt), device="cuda")
            if init is not None:
                o.copy_(torch.from_numpy(init))
            src = xd[off:off + n] if k == 3 else xd[:n]  # one misaligned input when off == 1
            xs.append(x[off:off + n] if k == 3 else x[:n])
            ds.append(xd)
            outs.append(o)
            inits.append(init)
            spec.append((op, dt, "gwv" if init is None else xr.mask_of("gwv") | xr.INIT_FROM_OUT,
                         src.data_ptr(), o.data_ptr()))
        n0 = xr.xr_launch_count()
        assert xr.xr_reduce_multi_at(spec, (n, 1, 1), torch.cuda.current_stream().cuda_stream) == 0
        torch.cuda.synchronize()
        assert xr.xr_launch_count() - n0 == 1
        for k, (op, dt) in enumerate(vars_):
            check(op, dt, (n, 1, 1), "gwv", outs[k].cpu().numpy(), xs[k], init=inits[k])


@pytest.mark.parametrize("op,dtype", [("+", "int32"), ("+", "fp32"), ("*", "fp64"), ("max", "fp32"), ("^", "int64"),
                                      ("&&", "int32"), ("min", "fp64"), ("||", "fp32")])
def test_rcluster_kernel(op, dtype, monkeypatch):
    """Small whole-array reductions (256 KiB - 4 MiB) on the opt-in cluster
    kernel (XR_CLUSTER=1): one thread-block cluster, gang tier through
    distributed shared memory (rank order, no ticket).  Ragged lengths, a
    misaligned start (scalar head), init."""
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_CLUSTER", "1")
    size = np.dtype(oracle.NP_DTYPES[dtype]).itemsize
    for nbytes in (256 << 10, (2 << 20) + 3 * size, 4 << 20):
        n = nbytes // size
        dims = (n, 1, 1)
        assert xr.xr_plan_describe(op, dtype, dims, "gwv", 256)["kernel"] == "rcluster"
        x = recipes.make(KIND[op], dims, 7, dtype, n % 1000)
        for offset in (0, 1):
            check(op, dtype, dims, "gwv", gpu_reduce(op, dtype, dims, "gwv", x, offset=offset), x)
        init = recipes.make("ints", (1, 1, 1), 1, dtype, 2)
        check(op, dtype, dims, "gwv", gpu_reduce(op, dtype, dims, "gwv", x, init=init), x, init=init)
    # the paper-style testsuite nest at gang+worker+vector (P1 closed form)
    lin = np.arange(64 * 64 * 128, dtype=np.int64).astype(np.int32)
    assert gpu_reduce("+", "int32", (64, 64, 128), "gwv", lin)[0] == -262144
