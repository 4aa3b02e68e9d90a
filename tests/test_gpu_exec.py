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


def _random_program(msize, nregs, t, seed, dt):
    """A random straight-line oblivious program: every op, random registers and
    addresses, many STORE -> LOAD pairs on the same address inside the executor's
    LOAD prefetch window (the host must mark those LOADs direct)."""
    rng = np.random.default_rng(seed)
    code = []
    for _ in range(t):
        op = int(rng.choice([0, 0, 0, 1, 1, 2, 3, 4, 5, 6, 7]))
        r = lambda: int(rng.integers(0, nregs))
        a = int(rng.integers(0, min(msize, 6))) if rng.random() < 0.5 else int(rng.integers(0, msize))
        if op == 0:
            code.append((0, r(), a, 0))
        elif op == 1:
            code.append((1, a, r(), 0))
        elif op == 7:
            v = int(rng.integers(-1000, 1000)) if dt == "int32" else \
                int(np.array([rng.standard_normal()], dtype=np.float32).view(np.int32)[0])
            code.append((7, r(), v, 0))
        else:
            code.append((op, r(), r(), r()))
    return np.asarray(code, dtype=np.int32).reshape(-1, 4)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("seed,t,msize", [(1, 40, 8), (2, 300, 16), (3, 1000, 12), (4, 5, 3), (5, 2000, 64)])
def test_executor_random_programs_match_oracle(dt, layout, seed, t, msize):
    # stresses the LOAD prefetch ring (exec.cu): loads of addresses stored a few instructions
    # earlier, fewer LOADs than ring slots, registers read before any write (they start at 0)
    nregs = 7
    prog = _random_program(msize, nregs, t, seed, dt)
    p = 300
    x = bulkgen.prefix_input(msize, p, seed=seed, dtype=dt, layout=layout)
    if dt == "float32":
        x = (x * 8).astype(np.float32)
    ref = oracle.bulk_execute(prog, x, layout)
    buf = torch.empty(prog.shape[0] * 16, dtype=torch.uint8, device=DEV)
    got = torch.from_numpy(x).to(DEV)
    bo.execute(prog, got, layout, prog_buf=buf)
    g = got.cpu().numpy()
    if dt == "float32":            # long random chains can overflow to inf and inf - inf: NaN payloads
        nan = np.isnan(g)          # are the one thing IEEE leaves to the implementation (x86 vs GPU)
        assert np.array_equal(nan, np.isnan(ref))
        g, ref = g[~nan], ref[~nan]
    assert np.array_equal(g.view(np.uint32), ref.view(np.uint32))


def test_executor_registers_start_at_zero():
    prog = np.array([[2, 0, 1, 2],            # r0 <- r1 + r2 (never written: 0 + 0)
                     [1, 0, 0, 0],            # b[0] <- r0
                     [1, 1, 5, 0]], dtype=np.int32)   # b[1] <- r5
    x = torch.full((64, 4), 7, dtype=torch.int32, device=DEV)
    bo.execute(prog, x, bo.ROW_WISE)
    assert torch.all(x[:, :2] == 0) and torch.all(x[:, 2:] == 7)
