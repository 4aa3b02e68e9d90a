"""Pins for the generic oblivious-program interpreter (NEXT-3, Theorem 2,
P:132-137) and the program builders: interpreting the written-out algorithms
must reproduce independent references -- the prefix-sum oracle, numpy's sort
(library routine) for the bitonic network, the Algorithm OPT oracle -- and the
recorded address trace must be input independent."""
import numpy as np
import pytest

import bulkgen
import oracle
from paper_conf_ipps_tanitni14_b200 import programs


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n", [1, 2, 7, 32, 100])
def test_prefix_program_equals_prefix_oracle(dt, n):
    x = bulkgen.prefix_input(n, 1, seed=n, dtype=dt)[0]
    P = programs.prefix_sums(n, dt)
    assert P.array().shape == (3 * n + 1, 4)
    got = oracle.execute(P.array(), x)
    assert np.array_equal(got.view(np.uint32), oracle.prefix_sums(x).view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n", [1, 2, 4, 16, 64, 256])
def test_bitonic_program_sorts(dt, n):
    for seed in range(3):
        x = bulkgen.prefix_input(n, 1, seed=seed, dtype=dt)[0]
        if dt == "int32" and seed == 2:
            x = (x % 5).astype(np.int32)                  # many ties
        got = oracle.execute(programs.bitonic_sort(n).array(), x)
        assert np.array_equal(got, np.sort(x))


def test_bitonic_program_size():
    n = 64
    P = programs.bitonic_sort(n)
    stages = 6 * 7 // 2                                    # log n (log n + 1) / 2
    assert P.array().shape[0] == 6 * stages * (n // 2)     # 6 instructions per comparator


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n", [3, 4, 5, 8, 12])
def test_opt_program_equals_opt_oracle(dt, n):
    P = programs.optimal_triangulation(n, dt)
    for h in range(3):
        c = bulkgen.tri_instances(n, [h], seed=50 + n, dtype=dt)[0]
        mem = np.zeros(P.msize, dtype=c.dtype)
        mem[: n * n] = c.ravel()
        got = oracle.execute(P.array(), mem)[programs.opt_result_address(n)]
        assert got.view(np.uint32) == np.asarray(oracle.opt(c)).view(np.uint32)


def test_trace_is_input_independent_and_matches_program():
    n = 16
    P = programs.bitonic_sort(n)
    a = bulkgen.prefix_input(n, 1, seed=1, dtype="int32")[0]
    b = bulkgen.prefix_input(n, 1, seed=2, dtype="int32")[0]
    ta, tb = oracle.execute_trace(P.array(), a), oracle.execute_trace(P.array(), b)
    assert np.array_equal(ta, tb)
    code = P.array()
    mem_ops = code[(code[:, 0] == 0) | (code[:, 0] == 1)]
    want = np.where(mem_ops[:, 0] == 0, mem_ops[:, 2], mem_ops[:, 1])
    assert np.array_equal(ta[:, 2], want)


@pytest.mark.parametrize("dt", ["int32", "float32"])
def test_bulk_layouts_agree(dt):
    n, p = 16, 11
    x = bulkgen.prefix_input(n, p, seed=3, dtype=dt)
    P = programs.bitonic_sort(n).array()
    r = oracle.bulk_execute(P, x, oracle.ROW_WISE)
    c = oracle.bulk_execute(P, np.ascontiguousarray(x.T), oracle.COLUMN_WISE)
    assert np.array_equal(r, c.T)
    assert np.array_equal(r, np.sort(x, axis=1))
