"""Pins for the N1 transform-reduce oracle: Monte Carlo
pi (Fig 13c) and the inner product (Fig 13b)."""
import math

import numpy as np
import pytest

import datagen
import oracle


@pytest.mark.parametrize("m", [4, 7, 10])
@pytest.mark.parametrize("dtype", ["fp32", "fp64"])
def test_disk_count_exact_on_dyadic_lattice(m, dtype):
    """x = i/2^m, y = j/2^m with |i|,|j| <= 2^m: products and the sum are exact in
    fp32 (i^2 + j^2 < 2^24), so the count equals the integer count of lattice
    points strictly inside the unit circle (Gauss circle problem, brute force)."""
    N = 1 << m
    i = np.arange(-N, N, dtype=np.int64)
    I, J = np.meshgrid(i, i, indexing="ij")
    expect = int(np.count_nonzero(I * I + J * J < N * N))
    x = (I / N).astype(oracle.NP_DTYPES[dtype]).reshape(-1)
    y = (J / N).astype(oracle.NP_DTYPES[dtype]).reshape(-1)
    got = oracle.transform_reduce("disk", dtype, (x.size, 1, 1), "g", x, y)
    assert got.tolist() == [expect]
    # per-row counts (mask V over rows of the lattice): each row i counts j with j^2 < N^2 - i^2
    rows = oracle.transform_reduce("disk", dtype, (2 * N, 1, 2 * N), "v", x, y)
    assert rows.tolist() == [int(np.count_nonzero(ii * ii + i * i < N * N)) for ii in i]


def test_disk_count_statistical_pi():
    """4m/n within 5 standard deviations of pi (P15) on U[-1,1) samples."""
    n = 1 << 22
    for dtype in ("fp32", "fp64"):
        x = datagen.uniform_float(11, n, -1.0, 1.0, oracle.NP_DTYPES[dtype])
        y = datagen.uniform_float(12, n, -1.0, 1.0, oracle.NP_DTYPES[dtype])
        m = int(oracle.transform_reduce("disk", dtype, (n, 1, 1), "g", x, y)[0])
        p = math.pi / 4
        assert abs(4 * m / n - math.pi) <= 5 * 4 * math.sqrt(p * (1 - p) / n)


def test_disk_boundary_and_init():
    # points exactly on the circle are NOT counted (strict <, @44029)
    x = np.array([1.0, 0.0, 0.6, -0.6, 0.0], np.float32)
    y = np.array([0.0, -1.0, 0.8, 0.0, 0.0], np.float32)
    # 0.6^2 + 0.8^2 rounds in fp32 to exactly 1.0 -> not counted; (-0.6, 0) and (0, 0) are
    assert oracle.transform_reduce("disk", "fp32", (5, 1, 1), "g", x, y).tolist() == [2]
    assert oracle.transform_reduce("disk", "fp32", (5, 1, 1), "g", x, y,
                                   init=np.array([40], np.int64)).tolist() == [42]


@pytest.mark.parametrize("dtype", ["int32", "int64", "fp32", "fp64"])
def test_dot_closed_forms(dtype):
    dt = oracle.NP_DTYPES[dtype]
    n = 1000
    k = np.arange(n).astype(dt)
    assert oracle.transform_reduce("dot", dtype, (n, 1, 1), "g", k, k)[0] == n * (n - 1) * (2 * n - 1) // 6
    ones = np.ones(n, dt)
    assert oracle.transform_reduce("dot", dtype, (n, 1, 1), "g", ones, ones)[0] == n
    a = np.tile(np.array([1, 0], dt), n // 2)
    b = np.tile(np.array([0, 1], dt), n // 2)
    assert oracle.transform_reduce("dot", dtype, (n, 1, 1), "g", a, b)[0] == 0
    # dot with ones == the '+' reduction, for every mask
    x = datagen.uniform_int(3, 6 * 7 * 8, -50, 50, np.int64).astype(dt)
    for lv in ["g", "w", "v", "gw", "gv", "wv", "gwv"]:
        d = oracle.transform_reduce("dot", dtype, (6, 7, 8), lv, x, np.ones_like(x))
        assert np.array_equal(d, oracle.reduce("+", dtype, (6, 7, 8), lv, x))


def test_dot_int32_wraps_and_fp_bound():
    x = np.array([2**16, 2**16, 3], np.int32)
    assert oracle.transform_reduce("dot", "int32", (3, 1, 1), "g", x, x)[0] == 9  # 2*2^32 + 9 mod 2^32
    x = datagen.uniform_float(5, 4096, -1.0, 1.0, np.float64)
    y = datagen.uniform_float(6, 4096, -1.0, 1.0, np.float64)
    got, S = oracle.transform_reduce("dot", "fp64", (4096, 1, 1), "g", x, y, want_abs=True)
    assert abs(got[0] - math.fsum((x * y).tolist())) <= 1e-15 * S[0]
    # matmul inner product (Fig 13b): C[i][j] = sum_k A[i][k] B[k][j] as rows of A . columns of B
    A = datagen.uniform_int(7, 5 * 9, -9, 9, np.int64).reshape(5, 9)
    B = datagen.uniform_int(8, 9 * 4, -9, 9, np.int64).reshape(9, 4)
    xs = np.repeat(A, 4, axis=0).reshape(-1)                # row i of A, for each j
    ys = np.tile(B.T, (5, 1)).reshape(-1)                    # column j of B, for each i
    C = oracle.transform_reduce("dot", "int64", (20, 1, 9), "v", xs, ys).reshape(5, 4)
    assert np.array_equal(C, A @ B)


def test_unsupported_and_invalid():
    x = np.zeros(4, np.int32)
    with pytest.raises(oracle.OracleError) as e:
        oracle.transform_reduce("disk", "int32", (4, 1, 1), "g", x, x)
    assert e.value.status == oracle.ERR_UNSUPPORTED
