"""CPU tests of host-side logic added in round 2:

- the chunk schedule of xr_reduce_host (xr_host_chunks, host only): chunks tile
  the input exactly once in order, every output block is written first by
  exactly one chunk, and reducing chunk by chunk with "init from out" for the
  later chunks of a block equals the oracle on the whole nest (integer ops,
  exact) -- the gang tier across chunks described in include/xreduce.h;
- the Python binding's nest / out validation;
- bench.py's rank launcher: --gpus N with fewer visible GPUs, or a WORLD_SIZE
  that differs from --gpus, exits with a clear error.
"""
import itertools
import os
import subprocess
import sys

import numpy as np
import pytest

import datagen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MASKS = ["g", "w", "v", "gw", "gv", "wv", "gwv"]


@pytest.fixture(scope="module")
def xr():
    import paper_conf_ppopp_xutycc14_b200 as m
    return m


def chunked_reference(op, dtype, dims, levels, x, cap, xr, init=None):
    """Replay xr_reduce_host's schedule with the ORACLE as the per-chunk
    reducer: first chunk of a block merges the caller's init (if any), later
    chunks use the block's current value as init."""
    n_out = oracle.out_count(dims, levels)
    out = np.zeros(n_out, dtype=oracle.NP_DTYPES[dtype]) if init is None else init.copy()
    size = x.itemsize
    for cd, in_off, out_off, first in xr.xr_host_chunks(dims, levels, dtype, cap):
        n = cd[0] * cd[1] * cd[2]
        k = oracle.out_count(cd, levels)
        seg = x[in_off:in_off + n]
        blk_init = None if (first and init is None) else out[out_off:out_off + k]
        out[out_off:out_off + k] = oracle.reduce(op, dtype, cd, levels, seg, init=blk_init)
    return out


@pytest.mark.parametrize("dims", [(7, 5, 3), (1, 9, 11), (13, 1, 6), (4, 6, 1), (3, 1, 1), (1, 1, 37)])
@pytest.mark.parametrize("cap_elems", [1, 2, 5, 17, 64, 10**6])
def test_host_chunks_tile_the_input(xr, dims, cap_elems):
    size = 4
    for lv in MASKS:
        chunks = xr.xr_host_chunks(dims, lv, "int32", cap_elems * size)
        total = dims[0] * dims[1] * dims[2]
        pos = 0
        for cd, in_off, out_off, first in chunks:
            assert in_off == pos, (lv, cd, in_off, pos)
            n = cd[0] * cd[1] * cd[2]
            assert n <= cap_elems, (cd, cap_elems)
            pos += n
        assert pos == total
        # every output element is covered, and each block has exactly one first writer
        n_out = oracle.out_count(dims, lv)
        firsts = np.zeros(n_out, dtype=np.int64)
        cover = np.zeros(n_out, dtype=np.int64)
        for cd, in_off, out_off, first in chunks:
            k = oracle.out_count(cd, lv)
            cover[out_off:out_off + k] += 1
            firsts[out_off:out_off + k] += int(first)
        assert cover.min() >= 1 and np.all(firsts == 1), (lv, cover, firsts)


@pytest.mark.parametrize("op,dtype", [("+", "int32"), ("*", "int64"), ("^", "int32"), ("max", "int64"),
                                      ("&&", "int32"), ("|", "int64")])
@pytest.mark.parametrize("dims,cap_elems", [((6, 5, 7), 9), ((1, 12, 10), 25), ((9, 1, 4), 3), ((5, 4, 3), 7)])
def test_chunked_schedule_equals_whole_nest(xr, op, dtype, dims, cap_elems):
    kinds = {"+": "ints", "*": "mul", "^": "bxor", "max": "maxmin", "&&": "land", "|": "bor"}
    from datagen import recipes
    for lv in MASKS:
        x = recipes.make(kinds[op], dims, oracle.mask_of(lv), dtype, 31)
        whole = oracle.reduce(op, dtype, dims, lv, x)
        got = chunked_reference(op, dtype, dims, lv, x, cap_elems * x.itemsize, xr)
        assert np.array_equal(got, whole), (op, dtype, dims, lv)
        init = datagen.uniform_int(5, oracle.out_count(dims, lv), -9, 9, oracle.NP_DTYPES[dtype])
        got = chunked_reference(op, dtype, dims, lv, x, cap_elems * x.itemsize, xr, init=init)
        assert np.array_equal(got, oracle.reduce(op, dtype, dims, lv, x, init=init)), (op, dims, lv, "init")


def test_host_chunks_validation(xr):
    with pytest.raises(xr.XReduceError):
        xr.xr_host_chunks((2, 2, 2), 0, "int32", 64)
    with pytest.raises(xr.XReduceError):
        xr.xr_host_chunks((2, 2, 2), "g", "int32", 0)
    assert xr.xr_host_chunks((0, 2, 2), "g", "int32", 64) == []


def test_python_nest_validation(xr):
    import torch
    t = torch.zeros(2, 3, 4, 5)
    assert xr._nest_of(t, None) == [6, 4, 5]          # leading dims flattened into n0
    assert xr._nest_of(torch.zeros(7), None) == [1, 1, 7]
    assert xr._nest_of(torch.zeros(3, 7), None) == [1, 3, 7]
    assert xr._nest_of(t, (12, 2, 5)) == [12, 2, 5]
    with pytest.raises(ValueError):
        xr._nest_of(t, (100, 1, 1))                  # more elements than the tensor
    with pytest.raises(ValueError):
        xr._nest_of(t, (2, 3))
    with pytest.raises(ValueError):
        xr.reduce(t, "+")                            # CPU tensor: no CPU fallback
    with pytest.raises(ValueError):
        xr._check_out(torch.zeros(3, dtype=torch.float64), torch.zeros(3), 3)   # dtype
    with pytest.raises(ValueError):
        xr._check_out(torch.zeros(2), torch.zeros(3), 3)                         # too small


def run_bench(args, env_extra=None):
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    env.update(env_extra or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True,
                          text=True, env=env, timeout=300)


def test_bench_gpus_without_enough_devices_fails_loudly():
    import torch
    if torch.cuda.device_count() >= 2:
        pytest.skip("this host has 2+ GPUs")
    r = run_bench(["--gpus", "2", "--steps", "1", "--warmup", "3"])
    assert r.returncode == 2, r.stderr
    assert "needs 2 visible GPUs" in r.stderr


def test_bench_world_size_mismatch_fails_loudly():
    r = run_bench(["--gpus", "2", "--steps", "1"], {"WORLD_SIZE": "4", "RANK": "0", "LOCAL_RANK": "0"})
    assert r.returncode == 2, r.stderr
    assert "WORLD_SIZE=4 but --gpus 2" in r.stderr
