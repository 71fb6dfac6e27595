"""The real NCCL path with a 1-rank communicator (one GPU is all this build can
get): xr_comm_get_unique_id / xr_comm_init over a torch.distributed group,
xr_reduce_sharded for every collective kind (the collective runs at every
world size, so ncclAllReduce with each op / dtype mapping, the in-place
ncclAllGather and the gather + fixed-order combine all execute here), the
sharded heat step (ncclAllReduce(max); with XR_FORCE_COLL also the grouped
ncclSend / ncclRecv halo exchange, to itself), xr_reduce_sharded_host and the
collective re-sync of xr_comm_set_fused -- checked against the oracle.
Multi-rank exchange semantics are covered by the single-device simulation
tests and the gloo world-2 tests."""
import os
import socket

import numpy as np
import pytest

import oracle
from datagen import recipes
from gpu_util import check

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def comm():
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_xutycc14_b200 as xr
    if not dist.is_initialized():
        with socket.socket() as s:
            s.bind(("127.0.0.1", 0))
            port = s.getsockname()[1]
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=0, world_size=1)
    torch.cuda.set_device(0)
    c = xr.Comm()
    yield c
    c.close()


@pytest.mark.parametrize("op,dtype,levels", [("+", "int64", "gwv"), ("max", "fp32", "g"), ("^", "int32", "gw"),
                                             ("&&", "fp64", "gv"), ("+", "fp32", "v"), ("*", "int32", "wv")])
def test_reduce_sharded_one_rank(comm, op, dtype, levels):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    dims = (40, 33, 65)
    kind = {"+": "ints", "max": "maxmin", "^": "bxor", "&&": "land", "*": "mul"}[op]
    x = recipes.make(kind, dims, oracle.mask_of(levels), dtype, 3)
    init = recipes.make("ints", (oracle.out_count(dims, levels), 1, 1), 1, dtype, 4)
    out = xr.reduce_sharded(torch.from_numpy(x).cuda(), comm, op, levels, nest_local=dims, init=init)
    torch.cuda.synchronize()
    check(op, dtype, dims, levels, out.cpu().numpy()[:init.size], x, init=init)


def test_heat_sharded_one_rank(comm):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    nj, ni, iters = 66, 130, 9
    T0 = oracle.heat_init(nj, ni)
    ref_T, ref_res = oracle.heat(nj, ni, iters, T0)
    slab = np.zeros((nj + 2, ni))
    slab[1:nj + 1] = T0.reshape(nj, ni)
    t1 = torch.from_numpy(slab.reshape(-1)).cuda()
    t2 = t1.clone()
    res = torch.zeros(iters, dtype=torch.float64, device="cuda")
    assert xr.xr_heat_run_sharded(nj, ni, iters, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), comm,
                                  torch.cuda.current_stream().cuda_stream) == 0
    torch.cuda.synchronize()
    assert res.cpu().tolist() == ref_res.tolist()
    fin = (t1 if iters % 2 == 0 else t2).cpu().numpy().reshape(nj + 2, ni)[1:nj + 1]
    assert np.array_equal(fin.view(np.uint64), ref_T.reshape(nj, ni).view(np.uint64))


def test_fused_exchange_one_rank(comm):
    """The real communicator with the fused exchange (1 rank: the mailbox is
    local) and with it disabled (NCCL): both equal the oracle."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    assert comm.query()["fused"]
    n = (1 << 22) + 7
    x = recipes.make("ints", (n, 1, 1), 7, "int64", 5)
    ref = oracle.reduce("+", "int64", (n, 1, 1), "gwv", x)
    xd = torch.from_numpy(x).cuda()
    for fused in (True, False, True):
        assert comm.set_fused(fused) == 0
        for _ in range(3):  # epochs advance, parity slots alternate
            out = xr.reduce_sharded(xd, comm, "+", "gwv", nest_local=(n, 1, 1))
            torch.cuda.synchronize()
            assert out.cpu().numpy()[:1].tolist() == ref.tolist()
    assert comm.query()["status"] == 0


def test_heat_sharded_forced_self_halo_exchange(comm, monkeypatch):
    """XR_FORCE_COLL: the 1-rank communicator exchanges its halo rows with
    itself, so the grouped ncclSend/ncclRecv call sites run on one GPU; NCCL
    matches the two self messages in order (halo row 0 <- owned row 1, halo
    row n+1 <- owned row n).  The owned rows stay bit-identical to the oracle."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_FORCE_COLL", "1")
    nj, ni, iters = 34, 66, 5
    T0 = oracle.heat_init(nj, ni)
    ref_T, ref_res = oracle.heat(nj, ni, iters, T0)
    slab = np.zeros((nj + 2, ni))
    slab[1:nj + 1] = T0.reshape(nj, ni)
    t1 = torch.from_numpy(slab.reshape(-1)).cuda()
    t2 = t1.clone()
    res = torch.zeros(iters, dtype=torch.float64, device="cuda")
    assert xr.xr_heat_run_sharded(nj, ni, iters, t1.data_ptr(), t2.data_ptr(), res.data_ptr(), comm,
                                  torch.cuda.current_stream().cuda_stream) == 0
    torch.cuda.synchronize()
    assert res.cpu().tolist() == ref_res.tolist()
    fin = (t1 if iters % 2 == 0 else t2).cpu().numpy().reshape(nj + 2, ni)
    assert np.array_equal(fin[1:nj + 1].view(np.uint64), ref_T.reshape(nj, ni).view(np.uint64))
    assert np.array_equal(fin[0], fin[1]) and np.array_equal(fin[nj + 1], fin[nj])


@pytest.mark.parametrize("op,dtype,levels", [("+", "int64", "gwv"), ("^", "int32", "g"), ("max", "fp64", "gv"),
                                             ("+", "int32", "wv"), ("||", "fp32", "gw")])
def test_reduce_sharded_host_one_rank(comm, monkeypatch, op, dtype, levels):
    """xr_reduce_sharded_host: pinned host slice -> chunked H2D + local
    reduction -> the collective -> host output, against the oracle."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    monkeypatch.setenv("XR_HOST_CHUNK_BYTES", "8192")
    dims = (40, 33, 65)
    kind = {"+": "ints", "max": "maxmin", "^": "bxor", "||": "lor"}[op]
    x = recipes.make(kind, dims, oracle.mask_of(levels), dtype, 13)
    xin = torch.from_numpy(x).pin_memory()
    n = oracle.out_count(dims, levels)
    init = recipes.make("ints", (n, 1, 1), 1, dtype, 4)
    out = init.copy()
    st = xr._lib.xr_reduce_sharded_host(xr.OPS[op], xr.DTYPES[dtype], xr._dims(dims),
                                        xr.mask_of(levels) | xr.INIT_FROM_OUT, xin.data_ptr(), out.ctypes.data,
                                        comm.handle, torch.cuda.current_stream().cuda_stream)
    assert st == 0, xr.xr_strerror(st)
    check(op, dtype, dims, levels, out, x, init=init)


def test_set_fused_is_collective_resync(comm):
    """Re-enabling the fused exchange re-aligns the epochs (NCCL max over the
    ranks) and clears the status word; the exchange keeps matching the
    oracle across toggles."""
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    n = (1 << 21) + 3
    x = recipes.make("ints", (n, 1, 1), 7, "int32", 8)
    ref = oracle.reduce("+", "int32", (n, 1, 1), "gwv", x)
    xd = torch.from_numpy(x).cuda()
    for _ in range(3):
        assert comm.set_fused(False) == 0
        assert comm.query()["fused"] is False
        assert comm.set_fused(True) == 0
        assert comm.query() == {"fused": True, "status": 0}
        out = xr.reduce_sharded(xd, comm, "+", "gwv", nest_local=(n, 1, 1))
        torch.cuda.synchronize()
        assert out.cpu().numpy()[:1].tolist() == ref.tolist()
