"""Multi-process (world_size 2, gloo, CPU) tests of the gang-sharded protocol's
host logic: the library's xr_shard_plan decides the exchange,
each rank reduces its contiguous gang slice (here with the oracle -- test
code), the collective runs over torch.distributed, and the result must equal
the unsharded oracle on the concatenated array (integers exactly, fp within
the C9/C10 bounds), with the initial value merged exactly once."""
import os
import socket

import numpy as np
import pytest

WORLD = 2


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


CASES = [
    # op, dtype, local_dims, levels, with_init
    ("+", "int32", (6, 5, 7), "g", True), ("+", "int64", (4, 3, 9), "gwv", True),
    ("*", "int32", (3, 4, 5), "gw", False), ("max", "fp32", (5, 6, 7), "gv", True),
    ("min", "fp64", (5, 6, 7), "g", False), ("&", "int64", (4, 5, 6), "gwv", True),
    ("|", "int32", (4, 5, 6), "gv", False), ("^", "int32", (7, 3, 5), "g", True),
    ("&&", "fp32", (6, 4, 5), "gw", False), ("||", "int64", (6, 4, 5), "gwv", True),
    ("+", "fp64", (8, 4, 16), "gwv", True), ("+", "int32", (6, 5, 7), "v", True),
    ("max", "int64", (4, 6, 8), "wv", False), ("^", "int64", (4, 6, 8), "w", True),
    ("*", "fp64", (4, 6, 8), "v", False),
]
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "&": "band", "|": "bor",
        "^": "bxor", "&&": "land", "||": "lor"}


def _worker(rank, port, results):
    import torch
    import torch.distributed as dist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    import oracle
    import paper_conf_ppopp_xutycc14_b200 as xr
    from datagen import recipes

    RED = {0: dist.ReduceOp.SUM, 1: dist.ReduceOp.PRODUCT, 2: dist.ReduceOp.MAX, 3: dist.ReduceOp.MIN}
    out = []
    for ci, (op, dtype, local, levels, with_init) in enumerate(CASES):
        mask = oracle.mask_of(levels)
        gdims = (local[0] * WORLD, local[1], local[2])
        n_loc = int(np.prod(local))
        full = recipes.make(KIND[op], gdims, mask, dtype, 500 + ci)
        mine = full[rank * n_loc:(rank + 1) * n_loc]
        # the datagen contract: a shard generated at its global start equals the slice
        shard = recipes.make(KIND[op], gdims, mask, dtype, 500 + ci, start=rank * n_loc, n=n_loc)
        assert np.array_equal(mine.view(np.uint8), shard.view(np.uint8))
        pmask = mask | (xr.INIT_FROM_OUT if with_init else 0)
        info = xr.xr_shard_plan(op, dtype, local, pmask, WORLD, rank)
        init = recipes.make("ints", (info["global_count"], 1, 1), 1, dtype, 77 + ci) if with_init else None
        seg = slice(info["out_offset"], info["out_offset"] + info["local_count"])
        local_init = init[seg] if (init is not None and info["local_init_from_out"]) else None
        part = oracle.reduce(op, dtype, local, levels, mine, init=local_init)
        t = torch.from_numpy(part.copy())
        coll = info["collective"]
        if coll == xr.COLL_ALLREDUCE:
            dist.all_reduce(t, op=RED[info["nccl_op"]])
            res = t.numpy()
        elif coll == xr.COLL_ALLGATHER_COMBINE:
            bufs = [torch.empty_like(t) for _ in range(WORLD)]
            dist.all_gather(bufs, t)
            g = np.stack([b.numpy() for b in bufs])  # rank-major, fixed order combine
            res = oracle.reduce(op, dtype, (WORLD, info["local_count"], 1), "g", g.reshape(-1))
        else:
            bufs = [torch.empty_like(t) for _ in range(WORLD)]
            dist.all_gather(bufs, t)
            res = np.concatenate([b.numpy() for b in bufs])
        ref, S = oracle.reduce(op, dtype, gdims, levels, full, init=init, want_abs=True)
        if dtype.startswith("fp") and op in ("+", "*"):
            tol = 1e-5 if dtype == "fp32" else 1e-12
            ok = bool(np.all(np.abs(res.astype(np.float64) - ref.astype(np.float64))
                             <= tol * np.maximum(S, np.abs(ref.astype(np.float64))) + 1e-300))
        else:
            ok = bool(np.array_equal(res.view(np.uint8), ref.view(np.uint8)))
        out.append((ci, ok, info["merge_init"]))
    results[rank] = out
    dist.destroy_process_group()


def test_sharded_protocol_gloo_world2():
    import torch.multiprocessing as mp
    mgr = mp.Manager()
    results = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(port, results), nprocs=WORLD, join=True)
    for rank in range(WORLD):
        for ci, ok, merged in results[rank]:
            assert ok, f"rank {rank} case {CASES[ci]}"
    # init merged exactly once when the gang level is reduced
    for ci, (op, dtype, local, levels, with_init) in enumerate(CASES):
        merges = [results[r][ci][2] for r in range(WORLD)]
        if "g" in levels and with_init:
            assert merges == [1, 0]
        elif with_init:
            assert merges == [1, 1]
