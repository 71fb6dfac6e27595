"""The all-cores OpenMP CPU baseline (cpubase/) agrees with the
oracle: bit-exact for integer, bitwise, logical and min/max ops; fp + and *
within the C9 / C10 bounds (the baseline accumulates in the data type, in a
thread-blocked order).  CPU only."""
import numpy as np
import pytest

import cpubase
import datagen
from datagen import recipes
import oracle

MASKS = ["g", "w", "v", "gw", "gv", "wv", "gwv"]
KIND = {"+": "ints", "*": "mul", "max": "maxmin", "min": "maxmin", "&": "band", "|": "bor",
        "^": "bxor", "&&": "land", "||": "lor"}
DTYPES = ["int32", "int64", "fp32", "fp64"]
PAIRS = [(op, dt) for op in KIND for dt in DTYPES if not (dt.startswith("fp") and op in "&|^")]


@pytest.mark.parametrize("op,dtype", PAIRS)
@pytest.mark.parametrize("dims", [(5, 7, 33), (37, 3, 129), (1, 1, 1000), (2, 300, 1), (64, 64, 128)])
def test_baseline_matches_oracle(op, dtype, dims):
    for levels in MASKS:
        mask = oracle.mask_of(levels)
        seed = datagen.case_seed(9, list(KIND).index(op), DTYPES.index(dtype), mask, 0)
        x = recipes.make(KIND[op], dims, mask, dtype, seed)
        for threads in (1, 3, 8):
            got = cpubase.reduce(op, dtype, dims, levels, x, threads=threads)
            if dtype.startswith("fp") and op in ("+", "*"):
                ref, S = oracle.reduce(op, dtype, dims, levels, x, want_abs=True)
                tau = 1e-5 if dtype == "fp32" else 1e-12
                bound = tau * S if op == "+" else tau * np.abs(ref.astype(np.float64)) + 1e-300
                assert np.all(np.abs(got.astype(np.float64) - ref.astype(np.float64)) <= bound), (levels, threads)
            else:
                ref = oracle.reduce(op, dtype, dims, levels, x)
                assert got.tobytes() == ref.tobytes(), (levels, threads)


@pytest.mark.parametrize("op", ["+", "max", "&&", "^"])
def test_baseline_init_merged_once(op):
    dims = (6, 5, 40)
    x = datagen.uniform_int(3, 1200, -50, 50, np.int64)
    for levels in MASKS:
        n = oracle.out_count(dims, levels)
        init = datagen.uniform_int(4, n, -9, 9, np.int64)
        got = cpubase.reduce(op, "int64", dims, levels, x, init=init, threads=4)
        ref = oracle.reduce(op, "int64", dims, levels, x, init=init)
        assert np.array_equal(got, ref), levels


def test_baseline_cfg1_closed_form():
    """cfg1 gwv over the linear index wraps to -262,144 (P1) on any thread count."""
    x = datagen.linear(64 * 64 * 128, np.int32)
    for t in (1, 2, 5, 8):
        assert cpubase.reduce("+", "int32", (64, 64, 128), "gwv", x, threads=t)[0] == -262144
