"""GPU parity: layout transpose, device input generator, checksums and the
host-buffer (end-to-end) entry points."""
import numpy as np
import pytest
import torch

import bulkgen
import oracle
import paper_conf_ipps_tanitni14_b200 as bo

pytestmark = pytest.mark.gpu
DEV = "cuda"


@pytest.mark.parametrize("rows,cols", [(1, 1), (4, 4), (3, 7), (64, 32), (65, 33), (128, 1024), (1000, 300),
                                       (4096, 36), (36, 4096), (2 ** 16 + 4, 20)])
def test_transpose_matches_oracle(rows, cols):
    x = bulkgen.prefix_input(cols, rows, seed=rows + cols, dtype="int32")
    got = bo.transpose(torch.from_numpy(x).to(DEV)).cpu().numpy()
    assert np.array_equal(got, oracle.transpose(x))


def test_transpose_unaligned_pointer():
    x = bulkgen.prefix_input(64, 64, seed=1, dtype="float32")
    buf = torch.zeros(x.size + 1, dtype=torch.float32, device=DEV)
    v = buf[1:].view(64, 64)
    v.copy_(torch.from_numpy(x))
    got = bo.transpose(v).cpu().numpy()
    assert np.array_equal(got, x.T)


def test_transpose_full_size_sampled():
    n, p = 1024, 2 ** 20
    x = bo.generate_prefix(n, p, 7, torch.int32, bo.ROW_WISE)
    t = bo.transpose(x)
    ids = torch.tensor([0, 1, 4095, 77777, p - 1], device=DEV)
    assert torch.equal(t[:, ids].T, x[ids])
    back = bo.transpose(t)
    assert torch.equal(back, x)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("kind", ["uniform", "ones", "arange", "smallint"])
def test_device_generator_equals_bulkgen(dt, layout, kind):
    n, p, h0 = 37, 53, 1000
    got = bo.generate_prefix(n, p, 9, getattr(torch, dt), layout, kind, h0=h0).cpu().numpy()
    ref = bulkgen.prefix_input(n, p, 9, dt, layout, kind, h0=h0)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("kind", ["chords", "full"])
@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE, bo.PACKED_ROW, bo.PACKED_COLUMN])
def test_device_tri_generator_equals_bulkgen(dt, layout, kind):
    for n, p, h0 in ((13, 29, 5), (3, 4, 0), (64, 9, 77)):
        got = bo.generate_tri(n, p, 3, getattr(torch, dt), layout, h0=h0, kind=kind).cpu().numpy()
        ref = bulkgen.tri_input(n, p, 3, dt, layout, h0=h0, kind=kind)
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_checksum_device_equals_host():
    x = bulkgen.prefix_input(40, 70, seed=5, dtype="float32")
    for layout in (bo.ROW_WISE, bo.COLUMN_WISE):
        xi = x if layout == bo.ROW_WISE else np.ascontiguousarray(x.T)
        d = int(bo.checksum(torch.from_numpy(xi).to(DEV), layout, h0=11).cpu().numpy().view(np.uint64)[0])
        assert d == bulkgen.checksum(xi, layout, h0=11)
    v = np.arange(100, dtype=np.int32)
    d = int(bo.checksum(torch.from_numpy(v).to(DEV), h0=3).cpu().numpy().view(np.uint64)[0])
    assert d == bulkgen.checksum(v, h0=3)


@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("variant", [bo.AUTO, bo.PS_NAIVE])
def test_prefix_host_entry_point(layout, variant):
    n, p = 256, 3000
    x = bulkgen.prefix_input(n, p, seed=6, dtype="float32", layout=layout)
    xh = torch.from_numpy(x).pin_memory()
    out = bo.prefix_sums_host(xh, layout, variant)
    assert np.array_equal(out.numpy().view(np.uint32), oracle.bulk_prefix_sums(x, layout).view(np.uint32))


def test_prefix_host_transposed_variant():
    n, p = 128, 1000
    x = bulkgen.prefix_input(n, p, seed=8, dtype="float32")
    out = bo.prefix_sums_host(torch.from_numpy(x).pin_memory(), bo.ROW_WISE, bo.PS_TRANSPOSED)
    assert np.array_equal(out.numpy().view(np.uint32), oracle.bulk_prefix_sums(x, 0).view(np.uint32))


@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE, bo.PACKED_ROW, bo.PACKED_COLUMN])
@pytest.mark.parametrize("variant", [bo.AUTO, bo.TRI_UMM_GLOBAL])
def test_tri_host_entry_point(layout, variant):
    n, p = 16, 2000
    for kind in ("chords", "full"):
        c = bulkgen.tri_input(n, p, seed=4, dtype="int32", layout=layout, kind=kind)
        out = bo.triangulation_host(torch.from_numpy(c).pin_memory(), layout, variant)
        assert np.array_equal(out.numpy(), oracle.bulk_opt(c, layout))


def test_launch_counter_counts_kernels():
    before = bo.launch_count()
    x = torch.zeros((16, 16), device=DEV)
    bo.prefix_sums(x, bo.ROW_WISE, bo.PS_TRANSPOSED)
    assert bo.launch_count() - before == 3          # transpose, scan, transpose


@pytest.mark.parametrize("n,p,variant", [(40, 1500, bo.AUTO), (40, 1500, bo.TRI_TILED_HALF),
                                         (80, 600, bo.TRI_TILED_GLOBAL), (80, 333, bo.TRI_TILED_GLOBAL8), (16, 700, bo.TRI_THREAD_REG)])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_tri_host_entry_point_chunked_variants(n, p, variant, layout):
    # several chunks in flight on the two internal streams; TILED_GLOBAL gives each stream its own scratch
    c = bulkgen.tri_input(n, p, seed=n + p, dtype="float32", layout=layout, kind="full")
    dt = bo.F32
    need = bo.triangulation_host_bytes(n, p, dt, layout, variant)
    assert need >= c.size * 4 + p * 4
    out = bo.triangulation_host(torch.from_numpy(c).pin_memory(), layout, variant)
    ref = oracle.bulk_opt(c, layout)
    assert np.array_equal(out.numpy().view(np.uint32), ref.view(np.uint32))
    short = torch.empty(need - 4, dtype=torch.uint8, device=DEV)
    with pytest.raises(bo.BulkError):
        bo.triangulation_host(torch.from_numpy(c).pin_memory(), layout, variant, device_buf=short)
