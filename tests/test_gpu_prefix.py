"""GPU parity: bulk prefix sums (every variant, both layouts, both dtypes)
against the CPU oracle, element by element; full-size PS-2 on sampled
instances.  Bar: bit-exact, except BO_PS_WARPSCAN fp32 (reassociated) which
is held to |gpu - oracle| <= 1e-5 * |oracle| (BASELINE.json north_star)."""
import numpy as np
import pytest
import torch

import bulkgen
import oracle
import paper_conf_ipps_tanitni14_b200 as bo

pytestmark = pytest.mark.gpu
DEV = "cuda"

ROW_VARIANTS = [bo.AUTO, bo.PS_FUSED_ROW, bo.PS_WARPSCAN, bo.PS_TRANSPOSED, bo.PS_NAIVE]
COL_VARIANTS = [bo.AUTO, bo.PS_ACROSS, bo.PS_NAIVE]
SHAPES = [(1, 1), (3, 5), (32, 1024), (33, 257), (128, 128), (1000, 300), (1024, 777), (4096, 129), (5, 4099),
          (100, 1)]


def _compare(got, ref, exact):
    if exact:
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))
    else:
        assert np.all(np.abs(got.astype(np.float64) - ref) <= 1e-5 * np.abs(ref.astype(np.float64)) + 1e-30)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("variant", ROW_VARIANTS)
@pytest.mark.parametrize("n,p", SHAPES)
def test_row_wise_matches_oracle(dt, variant, n, p):
    x = bulkgen.prefix_input(n, p, seed=n * 7 + p, dtype=dt)
    got = bo.prefix_sums(torch.from_numpy(x).to(DEV), bo.ROW_WISE, variant).cpu().numpy()
    ref = oracle.bulk_prefix_sums(x, oracle.ROW_WISE)
    _compare(got, ref, dt == "int32" or variant != bo.PS_WARPSCAN)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("variant", COL_VARIANTS)
@pytest.mark.parametrize("n,p", SHAPES)
def test_column_wise_matches_oracle(dt, variant, n, p):
    x = bulkgen.prefix_input(n, p, seed=n * 3 + p, dtype=dt, layout=bulkgen.COLUMN_WISE)
    got = bo.prefix_sums(torch.from_numpy(x).to(DEV), bo.COLUMN_WISE, variant).cpu().numpy()
    ref = oracle.bulk_prefix_sums(x, oracle.COLUMN_WISE)
    _compare(got, ref, True)


@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_in_place_and_unaligned(layout):
    n, p = 300, 256
    x = bulkgen.prefix_input(n, p, seed=4, dtype="float32", layout=layout)
    ref = oracle.bulk_prefix_sums(x, layout)
    t = torch.from_numpy(x).to(DEV)
    bo.prefix_sums(t, layout, out=t)                                    # the paper's in-place form
    assert np.array_equal(t.cpu().numpy().view(np.uint32), ref.view(np.uint32))
    # misaligned base pointer (offset by one element) forces the non-TMA / scalar paths
    buf = torch.zeros(x.size + 1, dtype=torch.float32, device=DEV)
    view = buf[1:].view(x.shape)
    view.copy_(torch.from_numpy(x))
    out = torch.empty(x.size + 1, dtype=torch.float32, device=DEV)[1:].view(x.shape)
    bo.prefix_sums(view, layout, out=out)
    assert np.array_equal(out.cpu().numpy().view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
def test_closed_forms_on_gpu(dt):
    n, p = 1024, 512
    ones = bo.generate_prefix(n, p, 0, getattr(torch, dt), bo.ROW_WISE, "ones")
    got = bo.prefix_sums(ones, bo.ROW_WISE).cpu().numpy()
    assert np.array_equal(got, np.broadcast_to(np.arange(1, n + 1, dtype=got.dtype), (p, n)))
    ar = bo.generate_prefix(n, p, 0, getattr(torch, dt), bo.COLUMN_WISE, "arange")
    got = bo.prefix_sums(ar, bo.COLUMN_WISE).cpu().numpy()
    i = np.arange(n, dtype=np.int64)
    assert np.array_equal(got.astype(np.int64), np.broadcast_to((i * (i + 1) // 2)[:, None], (n, p)))


def test_int32_wraparound():
    x = np.full((4, 64), 2 ** 31 - 1, dtype=np.int32)
    got = bo.prefix_sums(torch.from_numpy(x).to(DEV), bo.ROW_WISE).cpu().numpy()
    assert np.array_equal(got, oracle.bulk_prefix_sums(x, oracle.ROW_WISE))


def test_empty_is_noop():
    t = torch.zeros((0, 16), dtype=torch.float32, device=DEV)
    bo.prefix_sums(t, bo.ROW_WISE)
    t = torch.zeros((16, 0), dtype=torch.float32, device=DEV)
    bo.prefix_sums(t, bo.ROW_WISE)


def test_errors_raise():
    t = torch.zeros((8, 8), dtype=torch.float32, device=DEV)
    with pytest.raises(bo.BulkError):
        bo.prefix_sums(t, bo.ROW_WISE, bo.PS_ACROSS)
    with pytest.raises(bo.BulkError):
        bo.prefix_sums(t, bo.COLUMN_WISE, bo.PS_FUSED_ROW)


# --------------------------------------------------------- full size (PS-2)
def _sample_ids(p, k=48, seed=0):
    rng = np.random.default_rng(seed)
    ids = set(rng.integers(0, p, k).tolist()) | {0, 1, 127, 128, p - 129, p - 1}
    return np.array(sorted(ids))


@pytest.mark.parametrize("variant", [bo.AUTO, bo.PS_TRANSPOSED])
def test_ps2_full_size_row_wise_sampled(variant):
    n, p, seed = 1024, 2 ** 20, 2
    x = bo.generate_prefix(n, p, seed, torch.float32, bo.ROW_WISE)
    y = bo.prefix_sums(x, bo.ROW_WISE, variant)
    ids = _sample_ids(p)
    got = y[torch.from_numpy(ids).to(DEV)].cpu().numpy()
    inp = bulkgen.prefix_instances(n, ids, seed, "float32")
    assert np.array_equal(x[torch.from_numpy(ids).to(DEV)].cpu().numpy(), inp)   # device generator == bulkgen
    ref = oracle.bulk_prefix_sums(inp, oracle.ROW_WISE)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))
    # property at full size: the last column equals the total of each row computed
    # by the column-wise kernel on the transposed data
    yc = bo.prefix_sums(bo.transpose(x), bo.COLUMN_WISE)
    assert torch.equal(yc[-1], y[:, -1])


def test_ps2_full_size_column_wise_sampled():
    n, p, seed = 1024, 2 ** 20, 2
    x = bo.generate_prefix(n, p, seed, torch.float32, bo.COLUMN_WISE)
    y = bo.prefix_sums(x, bo.COLUMN_WISE)
    ids = _sample_ids(p, seed=1)
    got = y[:, torch.from_numpy(ids).to(DEV)].cpu().numpy().T
    ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(n, ids, seed, "float32"), oracle.ROW_WISE)
    assert np.array_equal(np.ascontiguousarray(got).view(np.uint32), ref.view(np.uint32))


def test_ps1_full_config_exact():
    n, p = 32, 1024
    for kind in ("uniform", "ones"):
        x = bulkgen.prefix_input(n, p, seed=1, dtype="int32", kind=kind)
        for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
            xi = x if layout == bo.ROW_WISE else np.ascontiguousarray(x.T)
            got = bo.prefix_sums(torch.from_numpy(xi).to(DEV), layout).cpu().numpy()
            assert np.array_equal(got, oracle.bulk_prefix_sums(xi, layout))


def test_max_size_64bit_indexing():
    # n*p = 2^32 elements (16 GiB in, 16 GiB out): every index past 2^31 must be 64-bit
    n, p, seed = 1024, 2 ** 22, 11
    x = bo.generate_prefix(n, p, seed, torch.float32, bo.ROW_WISE)
    y = bo.prefix_sums(x, bo.ROW_WISE)
    ids = np.array([0, 2 ** 21 - 1, 2 ** 21, 2 ** 22 - 129, p - 1])
    got = y[torch.from_numpy(ids).to(DEV)].cpu().numpy()
    ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(n, ids, seed, "float32"), oracle.ROW_WISE)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))
    del y
    xc = bo.transpose(x)
    del x
    yc = bo.prefix_sums(xc, bo.COLUMN_WISE)
    got = yc[:, torch.from_numpy(ids).to(DEV)].T.contiguous().cpu().numpy()
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n,p", [(100, 37892), (77, 40000), (64, 38000)])
def test_column_wise_tma_ring_ragged(dt, n, p):
    # shapes on the TMA column-wise path (p % 4 == 0, >= 2*128*SMs instances, n >= 64) whose last
    # 128-instance block and last 32-row chunk are partial: element by element against the oracle
    x = bulkgen.prefix_input(n, p, seed=n + p, dtype=dt, layout=bulkgen.COLUMN_WISE)
    got = bo.prefix_sums(torch.from_numpy(x).to(DEV), bo.COLUMN_WISE).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), oracle.bulk_prefix_sums(x, oracle.COLUMN_WISE).view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n,p", [(96, 1000), (1060, 333), (4100, 64), (128, 37887), (32, 40)])
def test_fused_row_32_instance_tiles_multi_box_stages(dt, n, p):
    # the 32-instance fused-row tiles carry 4 TMA boxes per ring stage: chunk counts that are not a
    # multiple of 4 (3, 34, 129 chunks), a ragged last tile, and a tile count below the SM count
    x = bulkgen.prefix_input(n, p, seed=n + 3 * p, dtype=dt)
    got = bo.prefix_sums(torch.from_numpy(x).to(DEV), bo.ROW_WISE, bo.PS_FUSED_ROW).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), oracle.bulk_prefix_sums(x, oracle.ROW_WISE).view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n,p", [(256, 32), (300, 36), (1000, 4100), (257, 996), (4096, 132), (2000, 37884)])
def test_column_wise_tma_ring_32_wide(dt, n, p):
    # the 32-instance column-block TMA ring (p % 4 == 0, p below 2*128*SMs, n >= 256): partial last
    # 32-instance block and partial last 64-row chunk, element by element against the oracle
    x = bulkgen.prefix_input(n, p, seed=n * 7 + p, dtype=dt, layout=bulkgen.COLUMN_WISE)
    got = bo.prefix_sums(torch.from_numpy(x).to(DEV), bo.COLUMN_WISE).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), oracle.bulk_prefix_sums(x, oracle.COLUMN_WISE).view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_every_small_n_auto(dt, layout):
    # every n = 1..200 through AUTO (fused-row TMA / smem, across vec4 / scalar), ragged p
    for n in range(1, 201):
        p = 61 + (n % 7) * 13
        x = bulkgen.prefix_input(n, p, seed=2000 + n, dtype=dt, layout=layout)
        ref = oracle.bulk_prefix_sums(x, layout)
        got = bo.prefix_sums(torch.from_numpy(x).to(DEV), layout).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), n
