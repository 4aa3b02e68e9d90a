"""CPU-side checks of the C-ABI library: it builds for sm_100a, loads, exports
every function include/bulkobl.h declares, and rejects bad arguments before
touching the GPU (validation happens before any CUDA call)."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_ipps_tanitni14_b200 as bo
from paper_conf_ipps_tanitni14_b200 import build as bld

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bulkobl.h")


@pytest.fixture(scope="module")
def L():
    bld.build()
    return bo.lib()


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(bulk_[a-z0-9_]+)\s*\(", text)))


def test_header_declares_the_survey_entry_points():
    names = declared_functions()
    for must in ("bulk_prefix_sums", "bulk_triangulation", "bulk_transpose", "bulk_last_error",
                 "bulk_triangulation_workspace"):
        assert must in names


def test_every_declared_symbol_is_exported(L):
    out = subprocess.check_output(["nm", "-D", "--defined-only", bo.LIB_PATH]).decode()
    exported = set(re.findall(r" T (bulk_\w+)", out))
    missing = [f for f in declared_functions() if f not in exported]
    assert not missing, missing
    for f in declared_functions():
        getattr(L, f)


def test_library_is_sm100a_code(L):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", bo.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_sass_uses_tma_and_viaddmnmx():
    sass = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-sass", bo.LIB_PATH]).decode()
    assert "UTMALDG" in sass and "UTMASTG" in sass          # cp.async.bulk.tensor load/store
    assert "VIADDMNMX" in sass                             # fused int32 add+min (Algorithm OPT)


def test_version_and_no_error(L):
    assert "sm_100a" in bo.version()
    assert bo.lib().bulk_last_error() == b""


def test_argument_validation_without_gpu(L):
    p = ctypes.c_void_p(16)  # never dereferenced: validation fails first
    assert L.bulk_prefix_sums(p, p, -1, 4, 0, 0, 0, None, 0, None) == -1
    assert b"n and p" in L.bulk_last_error()
    assert L.bulk_prefix_sums(p, p, 4, 4, 7, 0, 0, None, 0, None) == -1          # bad dtype
    assert L.bulk_prefix_sums(p, p, 4, 4, 0, 3, 0, None, 0, None) == -1          # bad layout
    assert L.bulk_prefix_sums(None, None, 4, 4, 0, 0, 0, None, 0, None) == -1    # NULL
    assert L.bulk_prefix_sums(p, p, 4, 4, 0, 0, 99, None, 0, None) == -1         # bad variant
    assert L.bulk_prefix_sums(p, p, 4, 4, 0, 0, bo.PS_ACROSS, None, 0, None) == -2   # needs column-wise
    assert L.bulk_prefix_sums(p, p, 4, 4, 0, 1, bo.PS_FUSED_ROW, None, 0, None) == -2
    # partial overlap
    assert L.bulk_prefix_sums(ctypes.c_void_p(4096), ctypes.c_void_p(4100), 4, 4, 0, 0, 0, None, 0, None) == -1
    assert L.bulk_prefix_sums(p, p, 0, 4, 0, 0, 0, None, 0, None) == 0            # empty: no-op
    assert L.bulk_prefix_sums(p, p, 2 ** 30, 2 ** 30, 0, 0, 0, None, 0, None) == -1  # n*p overflow
    # triangulation
    assert L.bulk_triangulation(p, p, 2, 4, 0, 0, 0, None, 0, None) == -1         # n < 3 (reading G23)
    assert L.bulk_triangulation(p, p, 5, -1, 0, 0, 0, None, 0, None) == -1
    assert L.bulk_triangulation(p, p, 64, 4, 0, 0, 77, None, 0, None) == -1
    assert L.bulk_triangulation(p, p, 64, 4, 0, 0, bo.TRI_UMM_GLOBAL, None, 0, None) == -1  # workspace
    assert b"workspace" in L.bulk_last_error()
    assert L.bulk_triangulation(p, p, 64, 0, 0, 0, 0, None, 0, None) == 0          # p = 0
    # transpose
    assert L.bulk_transpose(p, ctypes.c_void_p(1 << 20), 4, 4, 8, None) == -2
    assert L.bulk_transpose(p, p, 4, 4, 4, None) == -1                            # in place not allowed
    assert L.bulk_transpose(p, p, 0, 4, 4, None) == 0


def test_workspace_overlap_and_alignment_rejected_without_gpu(L):
    # a prefix workspace may share no byte with src or dst; TILED_GLOBAL's workspace
    # must be 16-byte aligned (both checked before any CUDA call)
    src, dst = ctypes.c_void_p(1 << 20), ctypes.c_void_p(2 << 20)
    n, p = 4, 4                                                   # 64 bytes each
    need = n * p * 4
    for ws in ((2 << 20) + 16, (2 << 20) - 16, (1 << 20) + 60, (1 << 20) - 60):
        assert L.bulk_prefix_sums(src, dst, n, p, 0, 0, bo.PS_TRANSPOSED, ctypes.c_void_p(ws), need, None) == -1
        assert b"workspace overlaps" in L.bulk_last_error()
    assert L.bulk_triangulation(src, dst, 100, 8, 1, 0, bo.TRI_TILED_GLOBAL, ctypes.c_void_p((3 << 20) + 4),
                                1 << 30, None) == -1
    assert b"16-byte aligned" in L.bulk_last_error()


def test_workspace_and_variant_queries(L):
    assert bo.triangulation_workspace(64, 1000, bo.F32, bo.COLUMN_WISE, bo.TRI_UMM_GLOBAL) == 63 * 63 * 1000 * 4
    assert bo.triangulation_workspace(64, 1000, bo.F32, bo.COLUMN_WISE, bo.TRI_SMEM_WARP) == 0
    assert bo.prefix_sums_workspace(1024, 100, bo.F32, bo.ROW_WISE, bo.PS_TRANSPOSED) == 1024 * 100 * 4
    assert bo.prefix_sums_workspace(1024, 100, bo.F32, bo.ROW_WISE) == 0
    assert bo.prefix_sums_variant(1024, 100, bo.F32, bo.ROW_WISE) == bo.PS_FUSED_ROW
    assert bo.prefix_sums_variant(1024, 100, bo.F32, bo.COLUMN_WISE) == bo.PS_ACROSS
    assert bo.prefix_sums_variant(32, 1024, bo.I32, bo.ROW_WISE) == bo.PS_WARPSCAN     # int32: exact, latency win
    assert bo.prefix_sums_variant(32, 2 ** 22, bo.I32, bo.ROW_WISE) == bo.PS_FUSED_ROW
    assert bo.triangulation_variant(16, 100, bo.I32, bo.ROW_WISE) == bo.TRI_THREAD_REG
    assert bo.triangulation_variant(64, 100, bo.F32, bo.ROW_WISE) == bo.TRI_TILED_HALF
    assert bo.triangulation_variant(40, 100, bo.F32, bo.ROW_WISE) == bo.TRI_TILED_QUARTER
    assert bo.triangulation_variant(100, 100, bo.F32, bo.ROW_WISE) == bo.TRI_TILED_GLOBAL
    assert bo.triangulation_variant(512, 100, bo.F32, bo.ROW_WISE) == bo.TRI_TILED_GLOBAL8


def test_binding_refuses_cpu_tensors(L):
    import torch
    with pytest.raises(ValueError):
        bo.prefix_sums(torch.zeros(4, 4))
    with pytest.raises(ValueError):
        bo.triangulation(torch.zeros(2, 5, 5))


def test_product_package_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_tanitni14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f), errors="replace").read()
                assert "import oracle" not in text and "from oracle" not in text, f
                assert "oracle.c" not in text and "liboracle" not in text, f


def test_execute_validates_program_on_host(L):
    import numpy as np
    p = ctypes.c_void_p(4096)           # 16-byte aligned, never dereferenced
    good = np.array([[0, 0, 3, 0], [1, 3, 0, 0]], dtype=np.int32)
    for bad in ([[0, 0, 8, 0]], [[0, 5, 0, 0]], [[9, 0, 0, 0]], [[2, 0, 1, 70]]):
        prog = np.array(bad, dtype=np.int32)
        assert L.bulk_execute(prog.ctypes.data, 1, p, 16, p, 8, 4, 0, 0, 4, None) == -1
        assert b"bad instruction 0" in L.bulk_last_error()
    assert L.bulk_execute(good.ctypes.data, 2, p, 16, p, 8, 4, 0, 0, 4, None) == -1   # program buffer too small
    assert L.bulk_execute(good.ctypes.data, 2, p, 32, p, 8, 4, 0, 0, 0, None) == -1   # nregs = 0
    assert L.bulk_execute(good.ctypes.data, 0, p, 32, p, 8, 4, 0, 0, 4, None) == 0    # empty program


def test_program_prepare_validates_on_host(L):
    import numpy as np
    p = ctypes.c_void_p(4096)
    h = ctypes.c_int64(7)
    for bad in ([[0, 0, 8, 0]], [[1, 0, 9, 0]], [[14, 0, 0, 0]]):     # internal opcodes are not accepted either
        prog = np.array(bad, dtype=np.int32)
        assert L.bulk_program_prepare(prog.ctypes.data, 1, 8, 4, p, 16, None, ctypes.byref(h)) == -1
        assert b"bad instruction 0" in L.bulk_last_error() and h.value == 0
    good = np.array([[0, 0, 3, 0], [1, 3, 0, 0]], dtype=np.int32)
    assert L.bulk_program_prepare(good.ctypes.data, 2, 8, 4, p, 16, None, ctypes.byref(h)) == -1   # buffer small
    assert L.bulk_program_prepare(good.ctypes.data, 2, 8, 4, p, 32, None, None) == -1               # NULL handle
    assert L.bulk_execute_prepared(123456, p, 8, 4, 0, 0, None) == -1
    assert b"unknown program handle" in L.bulk_last_error()
    assert L.bulk_program_release(123456) == -1
