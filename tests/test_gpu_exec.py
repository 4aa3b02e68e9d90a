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
    addresses, many STORE -> LOAD pairs on the same address a few instructions apart."""
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
@pytest.mark.parametrize("seed,t,msize", [(1, 40, 8), (2, 300, 16), (3, 1000, 12), (4, 5, 3), (5, 2000, 64),
                                          (6, 1500, 400), (7, 900, 131)])
def test_executor_random_programs_match_oracle(dt, layout, seed, t, msize):
    # loads of addresses stored a few instructions earlier, registers read before any
    # write (they start at 0)
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


def _fusable_program(msize, nregs, t, seed):
    """Random programs made of the executor's superinstruction shapes (exec.cu: the
    compare-exchange LOAD,LOAD,MIN,MAX,STORE,STORE and LOAD,OP,STORE), with register
    and address collisions drawn often -- shapes that must fuse (either MIN/MAX
    operand order, stores of any of the four registers, STORE over a loaded
    address, both LOADs of one address) and near misses that must not (a register
    shared between the loads and the results, MIN over a third register) -- mixed
    with random single instructions."""
    rng = np.random.default_rng(seed)
    r = lambda: int(rng.integers(0, nregs))
    a = lambda: int(rng.integers(0, min(msize, 4)))
    code = []
    while len(code) < t:
        k = rng.random()
        if k < 0.4:                                  # compare-exchange shape
            ra, rb, rn, rx = (int(v) for v in rng.permutation(nregs)[:4])
            if rng.random() < 0.2:                   # near miss: a collision
                rn, rx = rng.choice([ra, rb, rn]), rng.choice([ra, rb, rx, rn])
            y1, z1 = (ra, rb) if rng.random() < 0.5 else (rb, ra)
            y2, z2 = (ra, rb) if rng.random() < 0.5 else (rb, ra)
            if rng.random() < 0.1:
                z1 = r()
            q = lambda: int(rng.choice([ra, rb, rn, rx, r()]) if rng.random() < 0.9 else r())
            code += [(0, ra, a(), 0), (0, rb, a(), 0), (4, rn, y1, z1), (5, rx, y2, z2),
                     (1, a(), q(), 0), (1, a(), q(), 0)]
        elif k < 0.55:                               # a run of in-place comparators (CE2 groups)
            ra, rb, rn, rx = (int(v) for v in rng.permutation(nregs)[:4])
            for _ in range(int(rng.integers(1, 10))):
                A, B = (int(v) for v in rng.permutation(min(msize, 4))[:2])
                y1, z1 = (ra, rb) if rng.random() < 0.5 else (rb, ra)
                y2, z2 = (ra, rb) if rng.random() < 0.5 else (rb, ra)
                code += [(0, ra, A, 0), (0, rb, B, 0), (4, rn, y1, z1), (5, rx, y2, z2),
                         (1, A, rn, 0), (1, B, rx, 0)] if rng.random() < 0.5 else \
                        [(0, ra, A, 0), (0, rb, B, 0), (4, rn, y1, z1), (5, rx, y2, z2),
                         (1, B, rx, 0), (1, A, rn, 0)]
        elif k < 0.7:                                # a run of accumulate steps (ACC_ADD groups)
            acc, tmp = (int(v) for v in rng.permutation(nregs)[:2])
            for _ in range(int(rng.integers(1, 20))):
                yz = (acc, tmp) if rng.random() < 0.5 else (tmp, acc)
                code += [(0, tmp, a(), 0), (2, acc, *yz), (1, a(), acc, 0)]
        elif k < 0.8:                                # load-op-store shape, collisions likely
            op = int(rng.integers(2, 6))
            code += [(0, r(), a(), 0), (op, r(), r(), r()), (1, a(), r(), 0)]
        else:
            op = int(rng.choice([0, 1, 2, 3, 4, 5, 6]))
            code.append((op, r(), a(), 0) if op == 0 else (op, a(), r(), 0) if op == 1 else (op, r(), r(), r()))
    return np.asarray(code[:t], dtype=np.int32).reshape(-1, 4)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("seed,t,nregs", [(11, 60, 5), (12, 600, 6), (13, 3000, 8), (14, 7, 4), (15, 2000, 64)])
@pytest.mark.parametrize("msize", [9, 300])          # staged in shared memory / direct (exec_staged_smem)
def test_executor_superinstruction_shapes_match_oracle(dt, layout, seed, t, nregs, msize):
    prog = _fusable_program(msize, nregs, t, seed)
    x = bulkgen.prefix_input(msize, 257 if msize < 100 else 1000, seed=seed, dtype=dt, layout=layout)
    ref = oracle.bulk_execute(prog, x, layout)
    got = torch.from_numpy(x).to(DEV)
    bo.execute(prog, got, layout)
    g = got.cpu().numpy()
    if dt == "float32":
        nan = np.isnan(g)
        assert np.array_equal(nan, np.isnan(ref))
        g, ref = g[~nan], ref[~nan]
    assert np.array_equal(g.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_executor_captured_runs_unfused_program(layout):
    # under graph capture the caller's program is uploaded as it is (api.cu)
    n, p = 64, 300
    P = programs.bitonic_sort(n)
    x = bulkgen.prefix_input(n, p, seed=3, dtype="int32", layout=layout)
    ref = oracle.bulk_execute(P.array(), x, layout)
    buf = torch.from_numpy(x).to(DEV)
    work = buf.clone()
    prog_buf = torch.empty(P.array().shape[0] * 16, dtype=torch.uint8, device=DEV)
    host = torch.from_numpy(P.array().copy()).pin_memory().numpy()   # read by the copy node at replay
    g = bo.Captured(lambda s: (work.copy_(buf), bo.execute(host, work, layout, prog_buf=prog_buf, stream=s)))
    g.replay()
    torch.cuda.synchronize()
    assert np.array_equal(work.cpu().numpy(), ref)


def test_executor_alternating_shared_memory_sizes():
    # the staged kernel's shared-memory opt-in is a per-kernel maximum: a large launch
    # after a smaller one after a large one must still launch (api.cu ensure_dyn_smem)
    outs = []
    for msize in (120, 8, 120, 40, 120):
        P = programs.bitonic_sort(8)
        code = P.array().copy()
        x = bulkgen.prefix_input(msize, 200, seed=msize, dtype="int32", layout=bo.COLUMN_WISE)
        ref = oracle.bulk_execute(code, x, bo.COLUMN_WISE)
        got = bo.execute(code, torch.from_numpy(x).to(DEV), bo.COLUMN_WISE).cpu().numpy()   # nregs 64
        outs.append(np.array_equal(got, ref))
    assert all(outs)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("prog,n,p", [("prefix", 1024, 300), ("bitonic", 64, 1000), ("bitonic", 256, 130)])
def test_prepared_program_matches_oracle(dt, layout, prog, n, p):
    P = programs.prefix_sums(n, dt) if prog == "prefix" else programs.bitonic_sort(n)
    prep = bo.prepare(P, n)
    for seed in (1, 2):                                   # one preparation, several memories
        x = bulkgen.prefix_input(n, p, seed=seed, dtype=dt, layout=layout)
        ref = oracle.bulk_execute(P.array(), x, layout)
        got = bo.execute(prep, torch.from_numpy(x).to(DEV), layout).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.filterwarnings("ignore:The CUDA Graph is empty")       # the refused capture records nothing
def test_prepared_program_checks_msize_and_capture():
    P = programs.bitonic_sort(16)
    prep = bo.prepare(P, 16)
    with pytest.raises(bo.BulkError, match="msize"):
        bo.execute(prep, torch.zeros((17, 8), dtype=torch.int32, device=DEV), bo.COLUMN_WISE)
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with pytest.raises(bo.BulkError, match="capturing"):
        with torch.cuda.graph(g, stream=s):
            bo.prepare(P, 16, stream=s)


@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_prepared_program_in_captured_graph(layout):
    n, p = 64, 500
    P = programs.bitonic_sort(n)
    prep = bo.prepare(P, n)
    x = bulkgen.prefix_input(n, p, seed=8, dtype="float32", layout=layout)
    ref = oracle.bulk_execute(P.array(), x, layout)
    src = torch.from_numpy(x).to(DEV)
    work = torch.empty_like(src)
    g = bo.Captured(lambda s: (work.copy_(src), bo.execute(prep, work, layout, stream=s)))
    for _ in range(2):
        work.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert np.array_equal(work.cpu().numpy(), ref)


def _drifting_program(msize, nregs, t, seed):
    """Random programs with locality: addresses drawn from a 40-word range that
    drifts through the memory, so the executor cuts them into several shared-memory
    windows (exec.cu, WIN) with registers, loads and stores crossing window changes."""
    rng = np.random.default_rng(seed)
    code, base = [], 0
    r = lambda: int(rng.integers(0, nregs))
    while len(code) < t:
        base = min(base + int(rng.integers(0, 3)), msize - 40)
        a = lambda: base + int(rng.integers(0, 40))
        k = rng.random()
        if k < 0.3:
            A, B = (base + int(v) for v in rng.permutation(40)[:2])
            code += [(0, 0, A, 0), (0, 1, B, 0), (4, 2, 0, 1), (5, 3, 0, 1), (1, A, 2, 0), (1, B, 3, 0)]
        elif k < 0.5:
            code += [(0, 4, a(), 0), (2, 5, 5, 4), (1, a(), 5, 0)]
        else:
            op = int(rng.choice([0, 1, 2, 3, 4, 5, 6]))
            code.append((op, r(), a(), 0) if op == 0 else (op, a(), r(), 0) if op == 1 else (op, r(), r(), r()))
    return np.asarray(code[:t], dtype=np.int32).reshape(-1, 4)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("seed,t,msize,p", [(21, 3000, 500, 300), (22, 800, 200, 129), (23, 5000, 1000, 1000)])
def test_executor_windowed_programs_match_oracle(dt, layout, seed, t, msize, p):
    prog = _drifting_program(msize, 6, t, seed)
    x = bulkgen.prefix_input(msize, p, seed=seed, dtype=dt, layout=layout)
    ref = oracle.bulk_execute(prog, x, layout)
    for run in ("call", "prepared"):
        got = torch.from_numpy(x).to(DEV)
        bo.execute(prog if run == "call" else bo.prepare(prog, msize), got, layout)
        g = got.cpu().numpy()
        r = ref
        if dt == "float32":
            nan = np.isnan(g)
            assert np.array_equal(nan, np.isnan(r))
            g, r = g[~nan], r[~nan]
        assert np.array_equal(g.view(np.uint32), r.view(np.uint32)), run


# ---------------------------------------------------------------------------
# Compiled programs (bulk_program_compile, jit.cu): the straight-line kernels
# NVRTC builds from a prepared program, bit for bit against the oracle
# interpreter -- registers in memory (column-wise msize <= 128, row-wise <= 95
# through shared memory) and the streaming shape (column-wise, larger msize,
# loads grouped ahead of their block with store-to-load forwarding).
# ---------------------------------------------------------------------------
def _compiled_case(kind, msize, t, seed, dt):
    if kind == "random":
        return _random_program(msize, 7, t, seed, dt)
    if kind == "fusable":
        return _fusable_program(msize, 6, t, seed)
    if kind == "bitonic":
        return programs.bitonic_sort(msize).array()
    if kind == "opt":                                # Algorithm OPT written out (t = seed vertices)
        return programs.optimal_triangulation(seed, dt).array()
    return programs.prefix_sums(msize, dt).array()


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("kind,msize,t,seed", [("random", 8, 300, 21), ("random", 64, 2000, 22), ("random", 95, 1500, 23),
                                               ("random", 96, 900, 24), ("random", 130, 1500, 25),
                                               ("random", 400, 1500, 26), ("fusable", 9, 600, 27),
                                               ("fusable", 300, 800, 28), ("bitonic", 64, 0, 0), ("bitonic", 1, 0, 0),
                                               ("prefix", 33, 0, 0), ("prefix", 300, 0, 0),
                                               ("opt", programs.optimal_triangulation(8).msize, 0, 8),
                                               ("opt", programs.optimal_triangulation(12).msize, 0, 12)])
def test_compiled_program_matches_oracle(dt, layout, kind, msize, t, seed):
    prog = _compiled_case(kind, msize, t, seed, dt)
    prep = bo.prepare(prog, msize)
    compiled = prep.compile(getattr(torch, dt), layout)
    if layout == bo.COLUMN_WISE or msize <= 95:
        assert compiled
    elif kind in ("random", "opt"):                  # scattered addresses: no window reuse, not compiled
        assert not compiled
    else:                                            # row-wise windows: prefix / fusable programs
        assert compiled
    if compiled:
        assert "bo_prog" in prep.source(getattr(torch, dt), layout)
    for p in (301, 128, 1):
        x = bulkgen.prefix_input(msize, p, seed=seed + p, dtype=dt, layout=layout)
        if dt == "float32":
            x = (x * 8).astype(np.float32)
        ref = oracle.bulk_execute(prog, x, layout)
        g = bo.execute(prep, torch.from_numpy(x).to(DEV), layout).cpu().numpy()
        if dt == "float32":
            nan = np.isnan(g)
            assert np.array_equal(nan, np.isnan(ref))
            g, ref = g[~nan], ref[~nan]
        assert np.array_equal(g.view(np.uint32), ref.view(np.uint32)), (kind, msize, p)


def test_compiled_program_nan_and_signed_zero_semantics():
    # MIN / MAX are the header's comparisons, not fminf / fmaxf: with a NaN or -0.0 operand
    # the compiled kernel must pick exactly the operand the interpreter picks
    vals = np.array([np.nan, -0.0, 0.0, 1.0, -np.inf, np.inf, -1.0], dtype=np.float32)
    prog = []
    out = 0
    for i in range(len(vals)):
        for j in range(len(vals)):
            prog += [(0, 0, i, 0), (0, 1, j, 0), (4, 2, 0, 1), (5, 3, 0, 1), (3, 4, 0, 1),
                     (1, 7 + out, 2, 0), (1, 8 + out, 3, 0), (1, 9 + out, 4, 0)]
            out += 3
    prog = np.asarray(prog, dtype=np.int32)
    msize = 7 + out
    x = np.zeros((msize, 64), dtype=np.float32)
    x[:7] = vals[:, None]
    ref = oracle.bulk_execute(prog, x, bo.COLUMN_WISE)
    prep = bo.prepare(prog, msize)
    assert prep.compile(torch.float32, bo.COLUMN_WISE)
    g = bo.execute(prep, torch.from_numpy(x).to(DEV), bo.COLUMN_WISE).cpu().numpy()
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(g), nan)
    assert np.array_equal(g[~nan].view(np.uint32), ref[~nan].view(np.uint32))


def test_compiled_program_in_captured_graph():
    n, p = 64, 1000
    P = programs.bitonic_sort(n)
    prep = bo.prepare(P, n)
    assert prep.compile(torch.int32, bo.COLUMN_WISE)
    x = bulkgen.prefix_input(n, p, seed=5, dtype="int32", layout=bo.COLUMN_WISE)
    ref = oracle.bulk_execute(P.array(), x, bo.COLUMN_WISE)
    buf = torch.from_numpy(x).to(DEV)
    work = buf.clone()
    g = bo.Captured(lambda s: (work.copy_(buf), bo.execute(prep, work, bo.COLUMN_WISE, stream=s)))
    for _ in range(2):
        g.replay()
    torch.cuda.synchronize()
    assert np.array_equal(work.cpu().numpy(), ref)
