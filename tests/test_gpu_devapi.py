"""N4: the public device API (include/xreduce_device.cuh) fused into user
kernels -- the shared-memory-free gang tier under a kernel that reserves
200 KiB of shared memory, and block_reduce for segmented outputs -- checked
against the oracle (TEST module tests/devapi/devapi_test.cu)."""
import ctypes
import os

import numpy as np
import pytest

import oracle
from datagen import recipes
from gpu_util import check, torch_dt

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))
CASES = [("+", "int32"), ("^", "int32"), ("max", "int64"), ("&&", "int64"), ("+", "fp32"), ("min", "fp32"),
         ("+", "fp64"), ("*", "fp64")]
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "^": "bxor", "&&": "land"}


@pytest.fixture(scope="module")
def lib():
    so = os.path.join(HERE, "devapi", "libxr_devapi_test.so")
    assert os.path.exists(so), "built by __graft_entry__.build()"
    L = ctypes.CDLL(so)
    L.devapi_gmem.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                              ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_int]
    L.devapi_block.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                               ctypes.c_void_p]
    return L


@pytest.mark.parametrize("op,dtype", CASES)
def test_grid_reduce_gmem_no_shared_memory(lib, op, dtype):
    import torch
    for n, grid in [(1, 1), (1000, 3), (5_000_001, 148), (1 << 22, 296)]:
        x = recipes.make(KIND[op], (n, 1, 1), 1, dtype, n)
        xd = torch.from_numpy(x).cuda()
        ws = torch.zeros(grid * 8 + 1, dtype=torch.float64, device="cuda")      # >= warps (8 per CTA) x 8 B
        ticket = torch.zeros(1, dtype=torch.int32, device="cuda")
        init = recipes.make("ints", (1, 1, 1), 1, dtype, 5)
        out = torch.from_numpy(init.copy()).cuda()
        for rep in range(2):  # the ticket self-resets
            out.copy_(torch.from_numpy(init))
            assert lib.devapi_gmem(oracle.OPS[op], oracle.DTYPES[dtype], xd.data_ptr(), n, out.data_ptr(),
                                   ws.data_ptr(), ticket.data_ptr(), grid, 1) == 0
            check(op, dtype, (n, 1, 1), "g", out.cpu().numpy(), x, init=init)
        assert int(ticket.item()) == 0


@pytest.mark.parametrize("op,dtype", CASES)
def test_block_reduce_segments(lib, op, dtype):
    import torch
    nseg, seg = 777, 1031
    x = recipes.make(KIND[op], (nseg, 1, seg), 4, dtype, 9)
    out = torch.zeros(nseg, dtype=torch_dt(dtype), device="cuda")
    assert lib.devapi_block(oracle.OPS[op], oracle.DTYPES[dtype], torch.from_numpy(x).cuda().data_ptr(), nseg, seg,
                            out.data_ptr()) == 0
    check(op, dtype, (nseg, 1, seg), "v", out.cpu().numpy(), x)
