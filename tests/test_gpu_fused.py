"""The fused cross-GPU exchange (one kernel: local reduction + peer-mailbox
exchange, no NCCL launch).  Single device: nranks concurrent kernels on
separate streams run the real publish / spin / combine protocol
(xr_reduce_fused_sim); every rank must end with the same bits, equal to the
oracle on the concatenated array, with the init merged once."""
import numpy as np
import pytest

import oracle
from datagen import recipes
from gpu_util import check, torch_dt

pytestmark = pytest.mark.gpu
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "&": "band", "|": "bor", "^": "bxor",
        "&&": "land", "||": "lor"}


def run_fused(op, dtype, n_local, G, init=None):
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    gdims = (n_local * G, 1, 1)
    x = recipes.make(KIND[op], gdims, 7, dtype, n_local + G)
    xd = torch.from_numpy(x).cuda()
    shards = [xd[r * n_local:(r + 1) * n_local] for r in range(G)]
    outs = [torch.zeros(1, dtype=torch_dt(dtype), device="cuda") for _ in range(G)]
    mask = xr.GANG | xr.WORKER | xr.VECTOR
    if init is not None:
        outs[0].copy_(torch.from_numpy(init))  # rank 0 carries the initial value
        mask |= xr.INIT_FROM_OUT
    st = xr.xr_reduce_fused_sim(op, dtype, (n_local, 1, 1), mask, [s.data_ptr() for s in shards],
                                [o.data_ptr() for o in outs])
    return st, x, [o.cpu().numpy() for o in outs]


@pytest.mark.parametrize("G", [2, 3, 4, 8])
@pytest.mark.parametrize("op,dtype", [("+", "int64"), ("+", "fp32"), ("max", "fp64"), ("^", "int32"),
                                      ("&&", "fp32"), ("*", "int32"), ("min", "int32"), ("|", "int64")])
def test_fused_exchange_sim(G, op, dtype):
    for n_local in (1 << 16, 5_000_003, 1 << 23):  # register seg path, odd size, TMA stream path
        for with_init in (False, True):
            init = recipes.make("ints", (1, 1, 1), 1, dtype, 3) if with_init else None
            st, x, outs = run_fused(op, dtype, n_local, G, init)
            assert st == 0
            first = outs[0].view(np.uint8).tobytes()
            assert all(o.view(np.uint8).tobytes() == first for o in outs), "ranks disagree"
            check(op, dtype, (x.size, 1, 1), "gwv", outs[0], x, init=init)


def test_fused_exchange_unsupported_plan():
    import torch
    import paper_conf_ppopp_xutycc14_b200 as xr
    x = torch.ones(64, device="cuda")
    o = [torch.zeros(1, device="cuda") for _ in range(2)]
    # 32-element shards are planned on sub-warp groups, which cannot host the exchange
    assert xr.xr_reduce_fused_sim("+", "fp32", (32, 1, 1), 7, [x.data_ptr(), x[32:].data_ptr()],
                                  [t.data_ptr() for t in o]) == xr.ERR_UNSUPPORTED
