"""GPU parity at the paper's remaining experiment shapes (§V):
  * prefix sums of n = 32K (= 32768) floats at p = 8K (the largest p the
    paper ran at that n), row-wise and column-wise, our kernels and the paper's
    naive thread-per-instance kernels (K1/K2, the Fig. 11 pair);
  * optimal triangulation of 8-gons at p = 4M (= 4194304) (Fig. 12),
    row-wise and column-wise, our kernels and the paper's UMM kernels.
AUTO runs are checked on EVERY instance against the oracle (inputs from
bulkgen on the host, in chunks); the other variants on sampled instances plus
a full-size cross-check between the two arrangements.  Bit-exact throughout
(the fp32 variants here all keep the sequential association)."""
import os

import numpy as np
import pytest
import torch

import bulkgen
import oracle
import paper_conf_ipps_tanitni14_b200 as bo

pytestmark = pytest.mark.gpu
DEV = "cuda"
NTHREADS = os.cpu_count() or 1


def _ids(p, k=200, seed=0):
    rng = np.random.default_rng(seed)
    return np.array(sorted(set(rng.integers(0, p, k).tolist()) | {0, 1, 31, 32, 127, 128, p - 129, p - 1}))


# ----------------------------------------------------------- prefix n = 32K
N32K, P8K, SEED_PS = 32768, 8192, 21


@pytest.fixture(scope="module")
def ps32k():
    x = bo.generate_prefix(N32K, P8K, SEED_PS, torch.float32, bo.ROW_WISE)
    return x


def test_ps32k_row_wise_auto_every_instance(ps32k):
    y = bo.prefix_sums(ps32k, bo.ROW_WISE)
    torch.cuda.synchronize()
    step = 512
    for h0 in range(0, P8K, step):
        inp = bulkgen.prefix_input(N32K, step, SEED_PS, "float32", bulkgen.ROW_WISE, h0=h0)
        ref = oracle.bulk_prefix_sums(inp, oracle.ROW_WISE, nthreads=NTHREADS)
        got = y[h0:h0 + step].cpu().numpy()
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), h0


@pytest.mark.parametrize("variant", [bo.PS_NAIVE, bo.PS_FUSED_ROW, bo.PS_TRANSPOSED])
def test_ps32k_row_wise_variants_sampled(ps32k, variant):
    y = bo.prefix_sums(ps32k, bo.ROW_WISE, variant)
    ids = _ids(P8K)
    got = y[torch.from_numpy(ids).to(DEV)].cpu().numpy()
    ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(N32K, ids, SEED_PS, "float32"), oracle.ROW_WISE,
                                  nthreads=NTHREADS)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("variant", [bo.AUTO, bo.PS_ACROSS, bo.PS_NAIVE])
def test_ps32k_column_wise_matches_row_wise(ps32k, variant):
    # column-wise [n][p] input = the transpose of the row-wise one; every result must agree
    # with the row-wise AUTO result (itself checked on every instance above) and the oracle
    yr = bo.prefix_sums(ps32k, bo.ROW_WISE)
    xc = bo.transpose(ps32k)
    yc = bo.prefix_sums(xc, bo.COLUMN_WISE, variant)
    assert torch.equal(bo.transpose(yc).view(torch.int32), yr.view(torch.int32))
    ids = _ids(P8K, seed=1)
    got = yc[:, torch.from_numpy(ids).to(DEV)].T.contiguous().cpu().numpy()
    ref = oracle.bulk_prefix_sums(bulkgen.prefix_instances(N32K, ids, SEED_PS, "float32"), oracle.ROW_WISE,
                                  nthreads=NTHREADS)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


# ------------------------------------------------------ 8-gons at p = 4M
N8, P4M, SEED_TR = 8, 4 * 2 ** 20, 23


@pytest.mark.parametrize("dt", ["float32", "int32"])
def test_8gons_4m_row_wise_auto_every_instance(dt):
    c = bo.generate_tri(N8, P4M, SEED_TR, getattr(torch, dt), bo.ROW_WISE)
    out = bo.triangulation(c, bo.ROW_WISE).cpu().numpy()
    step = 2 ** 19
    for h0 in range(0, P4M, step):
        cin = bulkgen.tri_input(N8, step, SEED_TR, dt, bulkgen.ROW_WISE, h0=h0)
        ref = oracle.bulk_opt(cin, oracle.ROW_WISE, nthreads=NTHREADS)
        assert np.array_equal(out[h0:h0 + step].view(np.uint32), ref.view(np.uint32)), h0


@pytest.mark.parametrize("layout,variant", [(bo.ROW_WISE, bo.TRI_UMM_GLOBAL), (bo.COLUMN_WISE, bo.AUTO),
                                            (bo.COLUMN_WISE, bo.TRI_UMM_GLOBAL), (bo.ROW_WISE, bo.TRI_THREAD_REG),
                                            (bo.PACKED_COLUMN, bo.AUTO)])
def test_8gons_4m_variants_agree_with_auto(layout, variant):
    # every variant/arrangement on the same 4M instances gives the row-wise AUTO result
    # bit for bit (full size), and the oracle on sampled instances
    c = bo.generate_tri(N8, P4M, SEED_TR, torch.float32, bo.ROW_WISE)
    ref_all = bo.triangulation(c, bo.ROW_WISE)
    if layout == bo.ROW_WISE:
        ci = c
    else:
        del c
        ci = bo.generate_tri(N8, P4M, SEED_TR, torch.float32, layout)
    need = bo.triangulation_workspace(N8, P4M, bo.F32, layout, variant)
    ws = torch.empty(need, dtype=torch.uint8, device=DEV) if need else None
    got = bo.triangulation(ci, layout, variant, workspace=ws)
    assert torch.equal(got.view(torch.int32), ref_all.view(torch.int32))
    ids = _ids(P4M, k=1000, seed=2)
    ref = oracle.bulk_opt(bulkgen.tri_instances(N8, ids, SEED_TR, "float32"), oracle.ROW_WISE, nthreads=NTHREADS)
    assert np.array_equal(got.cpu().numpy()[ids].view(np.uint32), ref.view(np.uint32))
