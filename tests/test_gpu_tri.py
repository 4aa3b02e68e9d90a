"""GPU parity: bulk optimal triangulation (every variant, both layouts, both
dtypes) against the CPU oracle -- bit-exact (min is exact and each sum keeps
the association of Algorithm OPT).  Full TR-1 and TR-2 configs
are verified on every instance."""
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


def _variants(n):
    v = [bo.AUTO, bo.TRI_UMM_GLOBAL, bo.TRI_SMEM_WARP, bo.TRI_TILED_GLOBAL, bo.TRI_TILED_GLOBAL8]
    if n <= 18:
        v.append(bo.TRI_THREAD_REG)
    if 5 <= n <= 64:
        v += [bo.TRI_TILED, bo.TRI_TILED_HALF, bo.TRI_TILED_QUARTER]
    return v


def _supported(n, variant):
    if variant in (bo.TRI_TILED, bo.TRI_TILED_HALF, bo.TRI_TILED_QUARTER) and n > 64:
        return False
    if variant in (bo.TRI_TILED, bo.TRI_TILED_HALF, bo.TRI_TILED_QUARTER):
        try:
            bo.triangulation(torch.zeros((1, n, n), device=DEV), bo.ROW_WISE, bo.TRI_TILED)
        except bo.BulkError as e:
            if e.status == -2:
                return False
            raise
    return True


CASES = [(3, 5), (4, 33), (5, 64), (8, 100), (13, 257), (16, 300), (17, 64), (18, 40), (24, 100), (33, 64),
         (40, 70), (63, 33), (64, 130), (65, 20), (100, 9), (128, 4)]


LAYOUTS = [bo.ROW_WISE, bo.COLUMN_WISE, bo.PACKED_ROW, bo.PACKED_COLUMN]


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", LAYOUTS)
@pytest.mark.parametrize("n,p", CASES)
def test_all_variants_match_oracle(dt, layout, n, p):
    c = bulkgen.tri_input(n, p, seed=n + 100 * p, dtype=dt, layout=layout)
    ref = oracle.bulk_opt(c, layout, nthreads=NTHREADS)
    ct = torch.from_numpy(c).to(DEV)
    for v in _variants(n):
        if not _supported(n, v):
            continue
        got = bo.triangulation(ct, layout, v).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), (n, p, v)


def test_n3_is_zero_and_closed_forms():
    c = torch.zeros((10, 3, 3), dtype=torch.int32, device=DEV)
    assert torch.all(bo.triangulation(c) == 0)
    # uniform chord weight w -> (n-3) w for every n
    for n in (5, 16, 17, 40, 64):
        w = np.zeros((n, n), dtype=np.int32)
        for a in range(n):
            for b in range(a + 2, n):
                if not (a == 0 and b == n - 1):
                    w[a, b] = 5
        ct = torch.from_numpy(np.broadcast_to(w, (7, n, n)).copy()).to(DEV)
        for v in _variants(n):
            if _supported(n, v):
                assert torch.all(bo.triangulation(ct, bo.ROW_WISE, v) == (n - 3) * 5), (n, v)


def test_hand_worked_pentagon():
    c = np.zeros((5, 5), dtype=np.int32)
    for (a, b), w in {(0, 2): 7, (0, 3): 2, (1, 3): 5, (1, 4): 9, (2, 4): 4}.items():
        c[a, b] = w
    got = bo.triangulation(torch.from_numpy(c[None]).to(DEV)).cpu().numpy()
    assert got.tolist() == [7]      # tests/golden/pentagon_worked.txt


@pytest.mark.parametrize("layout", LAYOUTS)
def test_tr1_full_config(layout):
    n, p = 16, 65536
    c = bo.generate_tri(n, p, 3, torch.int32, layout)
    got = bo.triangulation(c, layout).cpu().numpy()
    ref = oracle.bulk_opt(bulkgen.tri_input(n, p, 3, "int32", layout), layout, nthreads=NTHREADS)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_tr2_full_config(layout):
    n, p = 64, 65536
    c = bo.generate_tri(n, p, 4, torch.float32, layout)
    got = bo.triangulation(c, layout).cpu().numpy()
    ids = np.arange(p) if NTHREADS >= 16 else np.unique(np.r_[np.arange(0, p, 16), p - 1])
    ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 4, "float32"), oracle.ROW_WISE, nthreads=NTHREADS)
    assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("variant", [bo.TRI_SMEM_WARP, bo.TRI_TILED, bo.TRI_TILED_HALF, bo.TRI_TILED_QUARTER,
                                     bo.TRI_TILED_GLOBAL, bo.TRI_TILED_GLOBAL8, bo.TRI_UMM_GLOBAL])
def test_tr2_variants_agree_full_size(variant):
    n, p = 64, 65536
    c = bo.generate_tri(n, p, 4, torch.float32, bo.ROW_WISE)
    if not _supported(n, variant):
        pytest.skip("variant not built")
    a = bo.triangulation(c, bo.ROW_WISE, variant)
    b = bo.triangulation(bo.transpose(c.view(p, n * n)).view(n, n, p), bo.COLUMN_WISE, variant)
    assert torch.equal(a.view(torch.int32), b.view(torch.int32))
    ids = np.arange(0, p, 997)
    ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 4, "float32"), oracle.ROW_WISE, nthreads=NTHREADS)
    assert np.array_equal(a.cpu().numpy()[ids].view(np.uint32), ref.view(np.uint32))


# ------------------------------------------------------------------ NEXT-1 chords
@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", LAYOUTS)
@pytest.mark.parametrize("n,p", [(3, 7), (4, 40), (5, 33), (8, 100), (13, 64), (16, 300), (17, 50), (33, 64),
                                 (61, 20), (64, 130)])
def test_chords_match_oracle(dt, layout, n, p):
    c = bulkgen.tri_input(n, p, seed=7 * n + p, dtype=dt, layout=layout)
    ref_v, ref_ch = oracle.bulk_opt_chords(c, layout)
    v, ch = bo.triangulation_chords(torch.from_numpy(c).to(DEV), layout)
    assert np.array_equal(v.cpu().numpy().view(np.uint32), ref_v.view(np.uint32))
    assert np.array_equal(ch.cpu().numpy(), ref_ch)


def test_chords_ties_take_the_first_k():
    # uniform weights: every triangulation is optimal; the chosen one is fixed by the tie-break
    n, p = 40, 8
    w = np.zeros((n, n), dtype=np.int32)
    for a in range(n):
        for b in range(a + 2, n):
            if not (a == 0 and b == n - 1):
                w[a, b] = 3
    c = np.broadcast_to(w, (p, n, n)).copy()
    ref_v, ref_ch = oracle.bulk_opt_chords(c, oracle.ROW_WISE)
    v, ch = bo.triangulation_chords(torch.from_numpy(c).to(DEV))
    assert np.array_equal(v.cpu().numpy(), ref_v) and np.array_equal(ch.cpu().numpy(), ref_ch)


def test_chords_tr2_full_size_sampled():
    n, p = 64, 65536
    c = bo.generate_tri(n, p, 4, torch.float32, bo.ROW_WISE)
    v, ch = bo.triangulation_chords(c)
    assert torch.equal(v.view(torch.int32), bo.triangulation(c).view(torch.int32))
    ids = np.unique(np.r_[np.arange(0, p, 509), p - 1])
    ref_v, ref_ch = oracle.bulk_opt_chords(bulkgen.tri_instances(n, ids, 4, "float32"), oracle.ROW_WISE)
    assert np.array_equal(ch.cpu().numpy()[ids], ref_ch)


# ------------------------------------------------ NEXT-2: the paper's large polygons
@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
@pytest.mark.parametrize("n,p", [(256, 5), (512, 3), (130, 20), (203, 7)])
@pytest.mark.parametrize("variant", [bo.AUTO, bo.TRI_TILED_GLOBAL, bo.TRI_TILED_GLOBAL8])
def test_large_polygons_match_oracle(dt, layout, n, p, variant):
    c = bulkgen.tri_input(n, p, seed=n + p, dtype=dt, layout=layout)
    ref = oracle.bulk_opt(c, layout, nthreads=NTHREADS)
    got = bo.triangulation(torch.from_numpy(c).to(DEV), layout, variant).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_global8_many_instances_per_cta():
    # p > #SMs: every CTA reuses its table slot for several instances (stale cells from the
    # previous instance must not leak into the next one)
    n, p = 72, 700
    c = bulkgen.tri_input(n, p, seed=11, dtype="float32")
    ref = oracle.bulk_opt(c, oracle.ROW_WISE, nthreads=NTHREADS)
    got = bo.triangulation(torch.from_numpy(c).to(DEV), bo.ROW_WISE, bo.TRI_TILED_GLOBAL8).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_512gon_paper_config_sampled():
    n, p = 512, 1024                     # the paper's largest 512-gon run
    c = bo.generate_tri(n, p, 7, torch.float32, bo.ROW_WISE)
    got = bo.triangulation(c).cpu().numpy()
    ids = np.array([0, 511, 1023])
    ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 7, "float32"), oracle.ROW_WISE, nthreads=NTHREADS)
    assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32))


def test_tr2_large_p_64bit_indexing():
    # p = 2^21 instances of dense 64x64 weights = 32 GiB: instance offsets past 2^31 words
    n, p, seed = 64, 2 ** 21, 12
    c = bo.generate_tri(n, p, seed, torch.float32, bo.ROW_WISE)
    got = bo.triangulation(c).cpu().numpy()
    ids = np.array([0, 2 ** 19 + 3, 2 ** 20 + 7, p - 1])
    ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, seed, "float32"), oracle.ROW_WISE, nthreads=NTHREADS)
    assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.ROW_WISE, bo.COLUMN_WISE])
def test_every_n_auto(dt, layout):
    # every polygon size 3..130 through AUTO (THREAD_REG, TILED_QUARTER, TILED_HALF, TILED_GLOBAL
    # and their ragged tails), p not a multiple of any tile width
    for n in range(3, 131):
        p = 37 + (n % 5)
        c = bulkgen.tri_input(n, p, seed=1000 + n, dtype=dt, layout=layout)
        ref = oracle.bulk_opt(c, layout, nthreads=NTHREADS)
        got = bo.triangulation(torch.from_numpy(c).to(DEV), layout).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), n


# ---------------------------------------------------------------------------
# Un-narrowed inputs ('full' kind, bulkgen): signed weights on every entry
# Algorithm OPT reads -- the root side c[0][n-1] included, which P:199 adds at
# i = 1, j = n-1 -- and poison (NaN, +-inf, +-FLT_MAX, -0, garbage int32) on
# every entry it never reads (sides, diagonal, lower triangle; P:212 stores
# only b - a >= 2).  Any kernel that drops the root term, or lets an unread
# entry into its table, fails here.
# ---------------------------------------------------------------------------
FULL_CASES = [(3, 9), (4, 33), (5, 40), (7, 65), (8, 100), (12, 50), (13, 129), (16, 300), (17, 64), (18, 40),
              (21, 35), (24, 100), (29, 33), (33, 64), (40, 70), (47, 20), (56, 19), (57, 17), (61, 33), (63, 33),
              (64, 130), (65, 20), (66, 9), (100, 9), (128, 4), (131, 3)]


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", LAYOUTS)
@pytest.mark.parametrize("n,p", FULL_CASES)
def test_full_inputs_every_variant_matches_oracle(dt, layout, n, p):
    c = bulkgen.tri_input(n, p, seed=5 * n + p, dtype=dt, layout=layout, kind="full")
    ref = oracle.bulk_opt(c, layout, nthreads=NTHREADS)
    ct = torch.from_numpy(c).to(DEV)
    for v in _variants(n):
        if not _supported(n, v):
            continue
        got = bo.triangulation(ct, layout, v).cpu().numpy()
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), (n, p, v)


@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", LAYOUTS)
@pytest.mark.parametrize("n,p", [(3, 7), (4, 40), (5, 33), (9, 64), (16, 300), (17, 50), (31, 40), (33, 64),
                                 (61, 20), (63, 21), (64, 130)])
def test_full_inputs_chords_match_oracle(dt, layout, n, p):
    c = bulkgen.tri_input(n, p, seed=3 * n + p, dtype=dt, layout=layout, kind="full")
    ref_v, ref_ch = oracle.bulk_opt_chords(c, layout)
    v, ch = bo.triangulation_chords(torch.from_numpy(c).to(DEV), layout)
    assert np.array_equal(v.cpu().numpy().view(np.uint32), ref_v.view(np.uint32))
    assert np.array_equal(ch.cpu().numpy(), ref_ch)


def test_full_inputs_root_side_is_added():
    # the same instances with c[0][n-1] zeroed: every GPU result moves by exactly the root weight
    for n, dt in ((16, torch.int32), (40, torch.int32), (64, torch.int32), (130, torch.int32)):
        c = bo.generate_tri(n, 500, 21, dt, bo.ROW_WISE, kind="full")
        d = c.clone()
        d[:, 0, n - 1] = 0
        for v in _variants(n):
            if _supported(n, v):
                got = bo.triangulation(c, bo.ROW_WISE, v).long()
                z = bo.triangulation(d, bo.ROW_WISE, v).long()
                assert torch.equal(got - z, c[:, 0, n - 1].long()), (n, v)


def test_full_inputs_unread_entries_are_never_read():
    # re-poisoning the unread entries with other values changes nothing, bit for bit
    for n in (7, 16, 33, 64, 80):
        c = bo.generate_tri(n, 700, 22, torch.float32, bo.ROW_WISE, kind="full")
        a_ = torch.arange(n, device=DEV)
        unread = (a_[None, :] - a_[:, None] < 2)
        d = c.clone()
        d[:, unread] = float("-inf")
        e = c.clone()
        e[:, unread] = float("nan")
        for v in _variants(n):
            if _supported(n, v):
                r = bo.triangulation(c, bo.ROW_WISE, v).view(torch.int32)
                assert torch.equal(r, bo.triangulation(d, bo.ROW_WISE, v).view(torch.int32)), (n, v)
                assert torch.equal(r, bo.triangulation(e, bo.ROW_WISE, v).view(torch.int32)), (n, v)


# Table-slot reuse: with p large enough every persistent CTA (tiled kernels) or
# workspace slot (CTA-per-instance kernels) runs several instances in turn, so
# cells left by instance h -- including the padding columns b >= n when n % 4 != 0
# -- are live in the table when instance h + stride starts.
@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("n,p", [(17, 200000), (18, 150000), (33, 60000), (41, 40000), (61, 12000), (63, 12000),
                                 (65, 1200), (130, 500)])
def test_multipass_table_reuse_full_inputs(dt, n, p):
    c = bo.generate_tri(n, p, 23 + n, getattr(torch, dt), bo.ROW_WISE, kind="full")
    ids = np.arange(p) if n <= 33 or NTHREADS >= 16 else np.unique(np.r_[np.arange(0, p, 7), p - 1])
    ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 23 + n, dt, kind="full"), oracle.ROW_WISE,
                          nthreads=NTHREADS)
    for v in _variants(n):
        if v == bo.TRI_UMM_GLOBAL and n > 64:
            continue                                    # (n-1)^2 p workspace; covered above at small p
        if _supported(n, v):
            got = bo.triangulation(c, bo.ROW_WISE, v).cpu().numpy()
            assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32)), (n, v)


@pytest.mark.parametrize("layout", LAYOUTS)
def test_full_inputs_tr1_tr2_shapes(layout):
    # the configs' shapes on un-narrowed inputs: TR-1 (int32 n=16) on every instance,
    # TR-2 (fp32 n=64) on every 8th instance + the last
    for n, p, dt, step in ((16, 65536, "int32", 1), (64, 65536, "float32", 8)):
        c = bo.generate_tri(n, p, 24, getattr(torch, dt), layout, kind="full")
        got = bo.triangulation(c, layout).cpu().numpy()
        ids = np.unique(np.r_[np.arange(0, p, step), p - 1])
        ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 24, dt, kind="full"), oracle.ROW_WISE,
                              nthreads=NTHREADS)
        assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32)), (n, layout)


# Column-wise weights through the CTA-cooperative whole-sector preload (tiled kernels with
# 8 or 16 consecutive instances per CTA batch, p % 8 == 0, 32-byte aligned weights; packed
# row-wise weights take the cooperative path at any p and alignment):
# every CTA runs several batches, p % 16 == 8 leaves a per-warp tail batch for the
# 16-instance CTAs, and an offset view (not 32-byte aligned) takes the per-warp path.
@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("layout", [bo.COLUMN_WISE, bo.PACKED_COLUMN, bo.PACKED_ROW])
@pytest.mark.parametrize("n,p", [(5, 40008), (8, 24000), (13, 16008), (17, 12000), (24, 9992), (33, 8008),
                                 (40, 6000), (61, 4008), (63, 4000), (64, 12008)])
def test_coop_column_preload_full_inputs(dt, layout, n, p):
    c = bulkgen.tri_input(n, p, seed=31 * n + p, dtype=dt, layout=layout, kind="full")
    ids = np.unique(np.r_[np.arange(0, p, 5), np.arange(p - 24, p)])
    ct = torch.from_numpy(c).to(DEV)
    ref = oracle.bulk_opt(bulkgen.tri_instances(n, ids, 31 * n + p, dt, kind="full"), oracle.ROW_WISE,
                          nthreads=NTHREADS)
    for v in [bo.AUTO, bo.TRI_TILED, bo.TRI_TILED_HALF, bo.TRI_TILED_QUARTER]:
        if _supported(n, v):
            got = bo.triangulation(ct, layout, v).cpu().numpy()
            assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32)), (n, v)
    # the same weights 4 bytes off a 32-byte boundary (per-warp preload path)
    buf = torch.empty(ct.numel() + 8, dtype=ct.dtype, device=DEV)
    off = buf[1:1 + ct.numel()].view(ct.shape)
    off.copy_(ct)
    got = bo.triangulation(off, layout, bo.TRI_TILED_HALF if n <= 64 else bo.AUTO).cpu().numpy()
    assert np.array_equal(got[ids].view(np.uint32), ref.view(np.uint32)), n
