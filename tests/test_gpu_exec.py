"""GPU parity for the generic bulk executor (NEXT-3): bit-exact against the
oracle interpreter on the same programs, both arrangements, both dtypes."""
import numpy as np
import pytest
import torch

import bulkgen
import oracle
import paper_conf_ipps_tanitni14_b200 as bo
from paper_conf_ipps_tanitni14_b200 import programs

pytestmark = pytest.mark.gpu
DEV = "cuda"


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("prog,n,p", [("prefix", 33, 300), ("bitonic", 64, 257), ("bitonic", 1, 5),
                                      ("prefix", 1, 1), ("bitonic", 256, 130)])
def test_executor_matches_oracle(dt, layout, prog, n, p):
    P = programs.prefix_sums(n, dt) if prog == "prefix" else programs.bitonic_sort(n)
    x = bulkgen.prefix_input(n, p, seed=n + p, dtype=dt, layout=layout)
    ref = oracle.bulk_execute(P.array(), x, layout)
    got = bo.execute(P, torch.from_numpy(x).to(DEV), layout).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_executor_runs_algorithm_opt(dt, layout):
    n, p = 10, 200
    P = programs.optimal_triangulation(n, dt)
    c = bulkgen.tri_input(n, p, seed=9, dtype=dt)                      # [p, n, n]
    mem = np.zeros((p, P.msize), dtype=c.dtype)
    mem[:, : n * n] = c.reshape(p, n * n)
    m = mem if layout == bo.ROW_WISE else np.ascontiguousarray(mem.T)
    got = bo.execute(P, torch.from_numpy(m).to(DEV), layout).cpu().numpy()
    res = got[:, programs.opt_result_address(n)] if layout == bo.ROW_WISE else got[programs.opt_result_address(n)]
    direct = bo.triangulation(torch.from_numpy(c).to(DEV)).cpu().numpy()
    assert np.array_equal(res.view(np.uint32), direct.view(np.uint32))
    assert np.array_equal(res.view(np.uint32), oracle.bulk_opt(c, oracle.ROW_WISE).view(np.uint32))


def test_executor_rejects_bad_program():
    x = torch.zeros((4, 8), dtype=torch.int32, device=DEV)
    bad = np.array([[0, 0, 8, 0]], dtype=np.int32)                      # address 8 >= msize 8
    with pytest.raises(bo.BulkError):
        bo.execute(bad, x, bo.ROW_WISE)
