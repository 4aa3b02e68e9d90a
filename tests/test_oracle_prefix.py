"""Pins for the prefix-sum oracle (Algorithm Prefix-sums).

Each test checks the oracle against something OTHER than itself: closed forms
typed by hand (tests/golden/prefix_closed_forms.txt), the defining identity
(first difference returns the input), linearity, exactness on integer-valued
floats, the library routine numpy.cumsum (a sequential accumulate, the same
left-to-right association as P:100), and an fp64 error bound.
"""
import numpy as np
import pytest

import bulkgen
import oracle
from conftest import read_golden


def _golden():
    return {row[0]: [int(x) for x in row[1:]] for row in read_golden("prefix_closed_forms.txt")}


@pytest.mark.parametrize("dt", [np.int32, np.float32])
def test_all_ones_gives_1_to_n(dt):
    g = _golden()["ones"]
    out = oracle.prefix_sums(np.ones(len(g), dtype=dt))
    assert out.tolist() == g
    big = oracle.prefix_sums(np.ones(1000, dtype=dt))
    assert np.array_equal(big, np.arange(1, 1001, dtype=dt))


@pytest.mark.parametrize("dt", [np.int32, np.float32])
def test_arange_gives_triangular_numbers(dt):
    g = _golden()["arange"]
    out = oracle.prefix_sums(np.arange(len(g), dtype=dt))
    assert out.tolist() == g
    n = 2000
    i = np.arange(n, dtype=np.int64)
    assert np.array_equal(oracle.prefix_sums(np.arange(n, dtype=dt)).astype(np.int64), i * (i + 1) // 2)


def test_int32_first_difference_returns_input_mod_2_32():
    x = bulkgen.prefix_input(777, 1, seed=11, dtype="int32")[0]
    y = oracle.prefix_sums(x)
    d = np.diff(np.concatenate([[0], y.view(np.uint32).astype(np.uint64)]).astype(np.uint64))
    assert np.array_equal((d & np.uint64(0xFFFFFFFF)).astype(np.uint32), x.view(np.uint32))


def test_int32_linearity_and_total_mod_2_32():
    a = bulkgen.prefix_input(513, 1, seed=1, dtype="int32")[0]
    b = bulkgen.prefix_input(513, 1, seed=2, dtype="int32")[0]
    s = (a.view(np.uint32) + b.view(np.uint32)).view(np.int32)
    lhs = oracle.prefix_sums(s).view(np.uint32)
    rhs = oracle.prefix_sums(a).view(np.uint32) + oracle.prefix_sums(b).view(np.uint32)
    assert np.array_equal(lhs, rhs)
    total = int(np.sum(a.astype(np.int64))) & 0xFFFFFFFF
    assert int(oracle.prefix_sums(a).view(np.uint32)[-1]) == total


def test_fp32_integer_valued_is_exact():
    # all partial sums < 2^24, so any association is exact: fp32 == int64 cumsum
    x = bulkgen.prefix_input(4096, 1, seed=5, dtype="float32", kind="smallint")[0]
    y = oracle.prefix_sums(x)
    assert np.array_equal(y.astype(np.int64), np.cumsum(x.astype(np.int64)))


def test_fp32_matches_sequential_library_accumulate():
    x = bulkgen.prefix_input(1024, 1, seed=2, dtype="float32")[0]
    y = oracle.prefix_sums(x)
    ref = np.add.accumulate(x, dtype=np.float32)   # sequential left-to-right in fp32
    assert np.array_equal(y.view(np.uint32), ref.view(np.uint32))


def test_fp32_within_sequential_rounding_bound_of_exact():
    n = 1024
    x = bulkgen.prefix_input(n, 1, seed=9, dtype="float32")[0]
    y = oracle.prefix_sums(x).astype(np.float64)
    exact = np.cumsum(x.astype(np.float64))
    # |err_i| <= i * u * sum_{q<=i} |x_q|  (u = 2^-24, sequential summation bound)
    i = np.arange(1, n + 1)
    assert np.all(np.abs(y - exact) <= i * 2.0 ** -24 * exact + 1e-30)


def test_empty_and_single():
    assert oracle.prefix_sums(np.zeros(0, dtype=np.int32)).size == 0
    assert oracle.prefix_sums(np.array([5], dtype=np.int32)).tolist() == [5]


@pytest.mark.parametrize("dt", ["int32", "float32"])
def test_bulk_row_and_column_arrangements_agree(dt):
    n, p = 37, 29
    row = bulkgen.prefix_input(n, p, seed=3, dtype=dt, layout=bulkgen.ROW_WISE)
    col = bulkgen.prefix_input(n, p, seed=3, dtype=dt, layout=bulkgen.COLUMN_WISE)
    assert np.array_equal(row.T, col)                     # P:122 vs P:124 addresses
    r = oracle.bulk_prefix_sums(row, oracle.ROW_WISE)
    c = oracle.bulk_prefix_sums(col, oracle.COLUMN_WISE, nthreads=3)
    assert np.array_equal(r.T.view(np.uint32), c.view(np.uint32))
    for j in range(p):
        assert np.array_equal(r[j].view(np.uint32), oracle.prefix_sums(row[j]).view(np.uint32))


def test_bulk_partial_range_leaves_others():
    n, p = 8, 10
    x = bulkgen.prefix_input(n, p, seed=4, dtype="int32")
    y = oracle.bulk_prefix_sums(x, oracle.ROW_WISE, h0=3, h1=7)
    assert np.array_equal(y[:3], x[:3]) and np.array_equal(y[7:], x[7:])
    assert np.array_equal(y[3:7], oracle.bulk_prefix_sums(x[3:7], oracle.ROW_WISE))
