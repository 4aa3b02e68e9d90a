"""Obliviousness and the UMM cost model, pinned on recorded address traces.

P:91 (Sec. III): an algorithm is oblivious if the address accessed at time i
is a fixed a(i), independent of the input.  P:104: for Algorithm Prefix-sums
a(2i) = a(2i+1) = i, t = 2n.  Algorithm OPT reads M[i,k],
M[k+1,j] per (i,j,k), then c[i-1,j], then writes M[i,j]: t(n) =
(n-1) + 2*C(n,3) + 2*C(n-1,2).  Lemma 1: in the bulk execution a
warp of w threads touches p... address groups per step: w groups row-wise,
1 group column-wise (UMM address groups A[j] of w cells).
"""
from math import comb

import numpy as np
import pytest

import bulkgen
import oracle


@pytest.mark.parametrize("dt", ["int32", "float32"])
def test_prefix_trace_closed_form_and_input_independence(dt):
    n = 50
    x1 = bulkgen.prefix_input(n, 1, seed=1, dtype=dt)[0]
    x2 = bulkgen.prefix_input(n, 1, seed=2, dtype=dt)[0]
    t1, t2 = oracle.prefix_trace(x1), oracle.prefix_trace(x2)
    assert len(t1) == 2 * n
    assert np.array_equal(t1, t2)
    i = np.arange(n)
    assert np.array_equal(t1[0::2, 2], i) and np.array_equal(t1[1::2, 2], i)  # a(2i)=a(2i+1)=i
    assert np.all(t1[0::2, 0] == 0) and np.all(t1[1::2, 0] == 1)              # read then write


@pytest.mark.parametrize("n", [3, 4, 8, 16, 20])
@pytest.mark.parametrize("dt", ["int32", "float32"])
def test_opt_trace_length_and_obliviousness(n, dt):
    c1 = bulkgen.tri_instances(n, [0], seed=1, dtype=dt)[0]
    c2 = bulkgen.tri_instances(n, [1], seed=2, dtype=dt)[0]
    t1, t2 = oracle.opt_trace(c1), oracle.opt_trace(c2)
    assert len(t1) == (n - 1) + 2 * comb(n, 3) + 2 * comb(n - 1, 2)
    assert np.array_equal(t1, t2)
    if n == 8:
        assert len(t1) == 161
    # the set of c entries read = {(a,b) : b - a >= 2}
    creads = t1[(t1[:, 1] == 1)]
    assert np.all(creads[:, 0] == 0)
    got = sorted(set(creads[:, 2].tolist()))
    want = sorted(a * n + b for a in range(n) for b in range(a + 2, n))
    assert got == want
    # M is written exactly once per cell of the upper triangle incl. diagonal
    mw = t1[(t1[:, 1] == 0) & (t1[:, 0] == 1)][:, 2]
    assert sorted(mw.tolist()) == sorted((i - 1) * (n - 1) + (j - 1)
                                         for i in range(1, n) for j in range(i, n))


def _groups_per_warp_step(addr_fn, trace_addr, p, w):
    """Max over warps of the number of distinct address groups (addr // w)
    touched when the p threads all access a(t) of their own instance."""
    worst = 0
    for a in trace_addr:
        addrs = np.array([addr_fn(int(a), j) for j in range(p)])
        for wi in range(p // w):
            worst = max(worst, len(set((addrs[wi * w:(wi + 1) * w] // w).tolist())))
    return worst


def test_lemma1_address_groups_row_vs_column():
    n, p, w = 32, 64, 32      # Lemma 1 assumes n >= w
    tr = oracle.prefix_trace(np.zeros(n, dtype=np.int32))[:, 2]
    row = _groups_per_warp_step(lambda a, j: j * n + a, tr, p, w)
    col = _groups_per_warp_step(lambda a, j: a * p + j, tr, p, w)
    assert row == w          # each warp step spans w groups ("p different groups" per step)
    assert col == 1          # coalesced: p/w groups per step, one per warp


def test_opt_bulk_column_wise_is_coalesced():
    n, p, w = 8, 64, 32       # row-wise stride (n-1)^2 = 49 >= w
    tr = oracle.opt_trace(np.zeros((n, n), dtype=np.int32))
    m_addr = tr[tr[:, 1] == 0][:, 2]
    col = _groups_per_warp_step(lambda a, h: a * p + h, m_addr, p, w)  # reading G7 column-wise
    row = _groups_per_warp_step(lambda a, h: h * (n - 1) ** 2 + a, m_addr, p, w)
    assert col == 1 and row == w
