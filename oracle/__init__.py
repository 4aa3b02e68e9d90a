"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs may import this package.  The product path
(paper_conf_ipps_tanitni14_b200) never imports it and shares no code with it.

Thin ctypes layer over oracle/oracle.c (plain C loops, one per instance, in
the paper's order: Algorithm Prefix-sums, Algorithm OPT P:174-200,
brute-force triangulation enumeration P:149-159, transpose P:122-124).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-std=c11", "-fPIC", "-shared",
          "-Wall", "-pthread"]

ROW_WISE, COLUMN_WISE, PACKED_ROW, PACKED_COLUMN = 0, 1, 2, 3
_DT = {"int32": 0, "float32": 1}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        i64, vp, i32 = ctypes.c_int64, ctypes.c_void_p, ctypes.c_int
        L.oracle_prefix_i32.argtypes = [vp, i64]
        L.oracle_prefix_f32.argtypes = [vp, i64]
        L.oracle_prefix_trace_i32.argtypes = [vp, i64, vp, i64]
        L.oracle_prefix_trace_i32.restype = i64
        L.oracle_prefix_trace_f32.argtypes = [vp, i64, vp, i64]
        L.oracle_prefix_trace_f32.restype = i64
        L.oracle_opt_i32.argtypes = [vp, i64, vp]
        L.oracle_opt_i32.restype = ctypes.c_int32
        L.oracle_opt_f32.argtypes = [vp, i64, vp]
        L.oracle_opt_f32.restype = ctypes.c_float
        L.oracle_opt_trace_i32.argtypes = [vp, i64, vp, i64]
        L.oracle_opt_trace_i32.restype = i64
        L.oracle_opt_trace_f32.argtypes = [vp, i64, vp, i64]
        L.oracle_opt_trace_f32.restype = i64
        L.oracle_brute_opt_f64.argtypes = [vp, i64, vp]
        L.oracle_brute_opt_f64.restype = ctypes.c_double
        L.oracle_transpose_u32.argtypes = [vp, vp, i64, i64]
        L.oracle_bulk_prefix.argtypes = [vp, i64, i64, i32, i32, i64, i64, i32]
        L.oracle_bulk_prefix.restype = i32
        L.oracle_bulk_opt.argtypes = [vp, vp, i64, i64, i32, i32, i64, i64, i32]
        L.oracle_bulk_opt.restype = i32
        L.oracle_opt_chords_i32.argtypes = [vp, i64, vp]
        L.oracle_opt_chords_i32.restype = ctypes.c_int32
        L.oracle_opt_chords_f32.argtypes = [vp, i64, vp]
        L.oracle_opt_chords_f32.restype = ctypes.c_float
        L.oracle_brute_opt_set_f64.argtypes = [vp, i64, vp]
        L.oracle_brute_opt_set_f64.restype = ctypes.c_double
        L.oracle_bulk_opt_chords.argtypes = [vp, vp, vp, i64, i64, i32, i32, i64, i64]
        L.oracle_bulk_opt_chords.restype = i32
        L.oracle_exec.argtypes = [vp, i64, vp, i32]
        L.oracle_exec.restype = i32
        L.oracle_exec_trace.argtypes = [vp, i64, vp, i32, vp, i64]
        L.oracle_exec_trace.restype = i64
        L.oracle_bulk_exec.argtypes = [vp, i64, vp, i64, i64, i32, i32]
        L.oracle_bulk_exec.restype = i32
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _dtname(a: np.ndarray) -> str:
    if a.dtype == np.int32:
        return "int32"
    if a.dtype == np.float32:
        return "float32"
    raise TypeError(f"oracle supports int32/float32, got {a.dtype}")


# ---------------------------------------------------------------- prefix sums
def prefix_sums(b: np.ndarray) -> np.ndarray:
    """Algorithm Prefix-sums on one array; returns a new array."""
    out = np.array(b, copy=True, order="C")
    fn = lib().oracle_prefix_i32 if _dtname(out) == "int32" else lib().oracle_prefix_f32
    fn(_ptr(out), out.size)
    return out


def prefix_trace(b: np.ndarray) -> np.ndarray:
    """Address trace [(kind, array, addr)] of one run (kind 0=read, 1=write)."""
    work = np.array(b, copy=True, order="C")
    cap = 2 * work.size
    ev = np.zeros((max(cap, 1), 3), dtype=np.int64)
    fn = lib().oracle_prefix_trace_i32 if _dtname(work) == "int32" else lib().oracle_prefix_trace_f32
    t = fn(_ptr(work), work.size, _ptr(ev), cap)
    assert t == cap, (t, cap)
    return ev[:t]


def bulk_prefix_sums(data: np.ndarray, layout: int, nthreads: int = 1,
                     h0: int = 0, h1: int | None = None) -> np.ndarray:
    """Parallel Algorithm Prefix-sums as p sequential runs.
    data: [p, n] (ROW_WISE) or [n, p] (COLUMN_WISE); returns a new array
    (instances outside [h0, h1) are returned unchanged)."""
    out = np.array(data, copy=True, order="C")
    if layout == ROW_WISE:
        p, n = out.shape
    else:
        n, p = out.shape
    h1 = p if h1 is None else h1
    rc = lib().oracle_bulk_prefix(_ptr(out), n, p, _DT[_dtname(out)], layout, h0, h1, nthreads)
    assert rc == 0
    return out


# ---------------------------------------------------------------------- OPT
def _tri_pn(c: np.ndarray, layout: int):
    """(p, n) of a weight array: [p,n,n] / [n,n,p] dense, [p,K] / [K,p] packed
    with K = (n-1)(n-2)/2 (the weights Algorithm OPT reads)."""
    if layout == ROW_WISE:
        return c.shape[0], c.shape[1]
    if layout == COLUMN_WISE:
        return c.shape[2], c.shape[0]
    K = c.shape[1] if layout == PACKED_ROW else c.shape[0]
    n = int(round((3 + (1 + 8 * K) ** 0.5) / 2))
    assert (n - 1) * (n - 2) // 2 == K, "bad packed size"
    return (c.shape[0] if layout == PACKED_ROW else c.shape[1]), n


def opt(c: np.ndarray, return_table: bool = False):
    """Algorithm OPT on one dense n x n weight matrix.
    Returns M[1, n-1]; with return_table also the (n-1)x(n-1) table
    (1-based M[i, j] at [i-1, j-1])."""
    c = np.ascontiguousarray(c)
    n = c.shape[0]
    assert c.shape == (n, n)
    M = np.zeros((max(n - 1, 1), max(n - 1, 1)), dtype=c.dtype)
    if _dtname(c) == "int32":
        v = lib().oracle_opt_i32(_ptr(c), n, _ptr(M))
    else:
        v = lib().oracle_opt_f32(_ptr(c), n, _ptr(M))
    v = c.dtype.type(v)
    return (v, M) if return_table else v


def opt_trace(c: np.ndarray) -> np.ndarray:
    c = np.ascontiguousarray(c)
    n = c.shape[0]
    cap = (n - 1) + 2 * (n * (n - 1) * (n - 2) // 6) + 2 * ((n - 1) * (n - 2) // 2)
    ev = np.zeros((max(cap, 1), 3), dtype=np.int64)
    fn = lib().oracle_opt_trace_i32 if _dtname(c) == "int32" else lib().oracle_opt_trace_f32
    t = fn(_ptr(c), n, _ptr(ev), cap)
    assert t == cap, (t, cap)
    return ev[:t]


def brute_opt(c: np.ndarray):
    """Minimum over ALL triangulations + c[0][n-1]; returns
    (value as float64, number of triangulations enumerated)."""
    w = np.ascontiguousarray(c, dtype=np.float64)
    n = w.shape[0]
    cnt = ctypes.c_int64(0)
    v = lib().oracle_brute_opt_f64(_ptr(w), n, ctypes.byref(cnt))
    return v, cnt.value


def bulk_opt(c: np.ndarray, layout: int, nthreads: int = 1,
             h0: int = 0, h1: int | None = None) -> np.ndarray:
    """Parallel Algorithm OPT as p sequential runs.
    c: [p, n, n] (ROW_WISE) or [n, n, p] (COLUMN_WISE); returns out[p]
    (entries outside [h0, h1) are 0)."""
    c = np.ascontiguousarray(c)
    p, n = _tri_pn(c, layout)
    h1 = p if h1 is None else h1
    out = np.zeros(p, dtype=c.dtype)
    rc = lib().oracle_bulk_opt(_ptr(c), _ptr(out), n, p, _DT[_dtname(c)], layout, h0, h1, nthreads)
    assert rc == 0
    return out


def opt_chords(c: np.ndarray):
    """Algorithm OPT with argmin bookkeeping (first minimising k as the
    strict '<' of P:196 keeps it) and the pre-order chord read-out.
    Returns (value, chords [n-3, 2] int16 of vertex pairs (a, b), a < b)."""
    c = np.ascontiguousarray(c)
    n = c.shape[0]
    ch = np.zeros((max(n - 3, 0), 2), dtype=np.int16)
    if _dtname(c) == "int32":
        v = lib().oracle_opt_chords_i32(_ptr(c), n, _ptr(ch))
    else:
        v = lib().oracle_opt_chords_f32(_ptr(c), n, _ptr(ch))
    return c.dtype.type(v), ch


def brute_opt_set(c: np.ndarray):
    """Brute-force optimum + the chord set of the first optimal triangulation
    found in lexicographic chord order; returns (value float64, chords [n-3, 2])."""
    w = np.ascontiguousarray(c, dtype=np.float64)
    n = w.shape[0]
    ch = np.zeros((max(n - 3, 0), 2), dtype=np.int16)
    v = lib().oracle_brute_opt_set_f64(_ptr(w), n, _ptr(ch))
    return v, ch


def bulk_opt_chords(c: np.ndarray, layout: int):
    """Parallel Algorithm OPT with chords for every instance: (out[p], chords[p, n-3, 2])."""
    c = np.ascontiguousarray(c)
    p, n = _tri_pn(c, layout)
    out = np.zeros(p, dtype=c.dtype)
    ch = np.zeros((p, max(n - 3, 0), 2), dtype=np.int16)
    rc = lib().oracle_bulk_opt_chords(_ptr(c), _ptr(out), _ptr(ch), n, p, _DT[_dtname(c)], layout, 0, p)
    assert rc == 0
    return out, ch


# ------------------------------------------------ generic oblivious programs
def execute(prog: np.ndarray, mem: np.ndarray) -> np.ndarray:
    """Interpret an oblivious program (int32 [t, 4]) on one instance memory."""
    prog = np.ascontiguousarray(prog, dtype=np.int32)
    out = np.array(mem, copy=True, order="C")
    rc = lib().oracle_exec(_ptr(prog), prog.shape[0], _ptr(out), _DT[_dtname(out)])
    assert rc == 0
    return out


def execute_trace(prog: np.ndarray, mem: np.ndarray) -> np.ndarray:
    prog = np.ascontiguousarray(prog, dtype=np.int32)
    work = np.array(mem, copy=True, order="C")
    cap = int(np.sum((prog[:, 0] == 0) | (prog[:, 0] == 1)))
    ev = np.zeros((max(cap, 1), 3), dtype=np.int64)
    t = lib().oracle_exec_trace(_ptr(prog), prog.shape[0], _ptr(work), _DT[_dtname(work)], _ptr(ev), cap)
    assert t == cap
    return ev[:t]


def bulk_execute(prog: np.ndarray, mem: np.ndarray, layout: int) -> np.ndarray:
    """Bulk execution (Thm 2): mem is [p, msize] row-wise or
    [msize, p] column-wise; returns the new memory."""
    prog = np.ascontiguousarray(prog, dtype=np.int32)
    out = np.array(mem, copy=True, order="C")
    if layout == ROW_WISE:
        p, msize = out.shape
    else:
        msize, p = out.shape
    rc = lib().oracle_bulk_exec(_ptr(prog), prog.shape[0], _ptr(out), msize, p, _DT[_dtname(out)], layout)
    assert rc == 0
    return out


# ----------------------------------------------------------------- transpose
def transpose(src: np.ndarray) -> np.ndarray:
    """dst[c*rows + r] = src[r*cols + c] for 4-byte elements."""
    src = np.ascontiguousarray(src)
    rows, cols = src.shape
    assert src.itemsize == 4
    dst = np.empty((cols, rows), dtype=src.dtype)
    lib().oracle_transpose_u32(_ptr(src), _ptr(dst), rows, cols)
    return dst
