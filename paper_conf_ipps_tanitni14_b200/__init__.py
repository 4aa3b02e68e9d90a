"""paper_conf_ipps_tanitni14_b200 -- Python binding of libbulkobl.so.

Bulk execution of oblivious sequential algorithms on B200 (Tani, Takafuji,
Nakano, Ito, IPDPS-W 2014): inclusive prefix sums (Algorithm Prefix-sums,
P:95-102), optimal convex-polygon triangulation (Algorithm OPT)
and the row-wise <-> column-wise transpose, each over p
independent instances.

This module only marshals arguments: torch supplies device memory and the
current CUDA stream, every step of the computation runs in the CUDA kernels
of libbulkobl.so (include/bulkobl.h).  There is no CPU fallback: if the
library is missing or a call fails, a BulkError is raised.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BULKOBL_LIB") or os.path.join(_HERE, "libbulkobl.so")   # override: A/B timing only

ROW_WISE, COLUMN_WISE, PACKED_ROW, PACKED_COLUMN = 0, 1, 2, 3
I32, F32 = 0, 1
AUTO = 0
PS_ACROSS, PS_WARPSCAN, PS_FUSED_ROW, PS_TRANSPOSED, PS_NAIVE = 1, 2, 3, 4, 5
TRI_UMM_GLOBAL, TRI_SMEM_WARP, TRI_THREAD_REG, TRI_TILED, TRI_TILED_HALF, TRI_TILED_GLOBAL = 16, 17, 18, 19, 20, 21
TRI_TILED_QUARTER = 22
TRI_TILED_GLOBAL8 = 23
VARIANT_NAMES = {
    AUTO: "auto", PS_ACROSS: "across", PS_WARPSCAN: "warpscan", PS_FUSED_ROW: "fused_row",
    PS_TRANSPOSED: "transposed", PS_NAIVE: "naive", TRI_UMM_GLOBAL: "umm_global",
    TRI_SMEM_WARP: "smem_warp", TRI_THREAD_REG: "thread_reg", TRI_TILED: "tiled", TRI_TILED_HALF: "tiled_half",
    TRI_TILED_GLOBAL: "tiled_global", TRI_TILED_QUARTER: "tiled_quarter",
    TRI_TILED_GLOBAL8: "tiled_global8",
}
KINDS = {"uniform": 0, "ones": 1, "arange": 2, "smallint": 3}
TR_KINDS = {"chords": 0, "full": 1}


class BulkError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"bulkobl status {status}: {msg}")
        self.status = status


_lib = None


def lib() -> ctypes.CDLL:
    """Load libbulkobl.so (built in-tree by __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python __graft_entry__.py build` "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        i64, vp, i32, sz, u64 = ctypes.c_int64, ctypes.c_void_p, ctypes.c_int, ctypes.c_size_t, ctypes.c_uint64
        sig = {
            "bulk_prefix_sums": ([vp, vp, i64, i64, i32, i32, i32, vp, sz, vp], i32),
            "bulk_prefix_sums_workspace": ([i64, i64, i32, i32, i32], sz),
            "bulk_triangulation": ([vp, vp, i64, i64, i32, i32, i32, vp, sz, vp], i32),
            "bulk_triangulation_workspace": ([i64, i64, i32, i32, i32], sz),
            "bulk_transpose": ([vp, vp, i64, i64, sz, vp], i32),
            "bulk_triangulation_chords": ([vp, vp, vp, i64, i64, i32, i32, vp], i32),
            "bulk_execute": ([vp, i64, vp, sz, vp, i64, i64, i32, i32, i32, vp], i32),
            "bulk_program_prepare": ([vp, i64, i64, i32, vp, sz, vp, ctypes.POINTER(i64)], i32),
            "bulk_execute_prepared": ([i64, vp, i64, i64, i32, i32, vp], i32),
            "bulk_program_compile": ([i64, i32, i32], i32),
            "bulk_program_source": ([i64, i32, i32, vp, sz, ctypes.POINTER(sz)], i32),
            "bulk_program_generate": ([vp, i64, i64, i32, i32, i32, vp, sz, ctypes.POINTER(sz)], i32),
            "bulk_program_release": ([i64], i32),
            "bulk_prefix_sums_host": ([vp, vp, i64, i64, i32, i32, i32, vp, sz, vp], i32),
            "bulk_triangulation_host": ([vp, vp, i64, i64, i32, i32, i32, vp, sz, vp], i32),
            "bulk_prefix_sums_host_bytes": ([i64, i64, i32, i32, i32], sz),
            "bulk_triangulation_host_bytes": ([i64, i64, i32, i32, i32], sz),
            "bulk_generate_prefix": ([vp, i64, i64, i64, u64, i32, i32, i32, vp], i32),
            "bulk_generate_tri": ([vp, i64, i64, i64, u64, i32, i32, i32, vp], i32),
            "bulk_checksum": ([vp, i64, i64, i64, i32, vp, vp], i32),
            "bulk_last_error": ([], ctypes.c_char_p),
            "bulk_prefix_sums_variant": ([i64, i64, i32, i32, i32, vp, vp], i32),
            "bulk_triangulation_variant": ([i64, i64, i32, i32, i32], i32),
            "bulk_launch_count": ([], u64),
            "bulk_version": ([], ctypes.c_char_p),
        }
        for name, (args, res) in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def _check(rc: int):
    if rc != 0:
        raise BulkError(rc, lib().bulk_last_error().decode())


_DTYPES = {torch.int32: 0, torch.float32: 1, "int32": 0, "float32": 1}


def _dtype_code(t: torch.Tensor) -> int:
    if t.dtype == torch.int32:
        return I32
    if t.dtype == torch.float32:
        return F32
    raise TypeError(f"bulkobl supports int32 and float32, got {t.dtype}")


_raw_stream = getattr(torch._C, "_cuda_getCurrentRawStream", None)


def _stream(stream=None, t: torch.Tensor | None = None) -> int:
    """cudaStream_t to launch on: `stream`, else the current stream of t's device
    (the raw-handle query: torch.cuda.current_stream() builds a Python object
    and costs ~5 us per call, half of a small call's host time)."""
    if stream is None and _raw_stream is not None and t is not None and t.is_cuda:
        return _raw_stream(t.device.index)
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


def _need_cuda(*ts):
    for t in ts:
        if not t.is_cuda:
            raise ValueError("device entry points need CUDA tensors (use *_host for host buffers)")
        if not t.is_contiguous():
            raise ValueError("tensors must be contiguous")


def _check_out(out: torch.Tensor, like: torch.Tensor, shape, what: str = "out"):
    """The C ABI cannot see buffer sizes: a caller-supplied output must be a
    contiguous CUDA tensor on the input's device, of its dtype and `shape`."""
    _need_cuda(out)
    if out.device != like.device or out.dtype != like.dtype or tuple(out.shape) != tuple(shape):
        raise ValueError(f"{what} must be a {like.dtype} tensor of shape {tuple(shape)} on {like.device}")


def _check_workspace(ws: torch.Tensor, like: torch.Tensor):
    _need_cuda(ws)
    if ws.device != like.device:
        raise ValueError(f"workspace must be on {like.device}")


def _shape_np(t: torch.Tensor, layout: int):
    if t.dim() != 2:
        raise ValueError("prefix sums take a 2-D tensor: [p, n] row-wise or [n, p] column-wise")
    return (t.shape[1], t.shape[0]) if layout == ROW_WISE else (t.shape[0], t.shape[1])


# ------------------------------------------------------------------ prefix
def prefix_sums_workspace(n: int, p: int, dtype: int, layout: int, variant: int = AUTO) -> int:
    return int(lib().bulk_prefix_sums_workspace(n, p, dtype, layout, variant))


def prefix_sums(x: torch.Tensor, layout: int = ROW_WISE, variant: int = AUTO, out: torch.Tensor | None = None,
                workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Inclusive prefix sums of every instance.  x is [p, n]
    (ROW_WISE) or [n, p] (COLUMN_WISE); out may be x (in place)."""
    _need_cuda(x)
    n, p = _shape_np(x, layout)
    dt = _dtype_code(x)
    if out is None:
        out = torch.empty_like(x)
    else:
        _check_out(out, x, x.shape)
    # only the explicit-transpose variant uses a workspace (AUTO never resolves to it):
    # skip the query, a ctypes round trip, on the hot small-call path
    need = prefix_sums_workspace(n, p, dt, layout, variant) if variant == PS_TRANSPOSED else 0
    wptr, wbytes = None, 0
    if need:
        if workspace is None:
            workspace = torch.empty(need, dtype=torch.uint8, device=x.device)
        _check_workspace(workspace, x)
        wptr, wbytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    _check(lib().bulk_prefix_sums(x.data_ptr(), out.data_ptr(), n, p, dt, layout, variant, wptr, wbytes,
                                  _stream(stream, x)))
    return out


def prefix_sums_variant(n: int, p: int, dtype: int, layout: int, variant: int = AUTO) -> int:
    return int(lib().bulk_prefix_sums_variant(n, p, dtype, layout, variant, None, None))


def prefix_sums_host_bytes(n: int, p: int, dtype: int, layout: int = ROW_WISE, variant: int = AUTO) -> int:
    """Device buffer size bulk_prefix_sums_host needs (data + per-stream workspace)."""
    return int(lib().bulk_prefix_sums_host_bytes(n, p, dtype, layout, variant))


def triangulation_host_bytes(n: int, p: int, dtype: int, layout: int = ROW_WISE, variant: int = AUTO) -> int:
    """Device buffer size bulk_triangulation_host needs (weights + output + workspace)."""
    return int(lib().bulk_triangulation_host_bytes(n, p, dtype, layout, variant))


def prefix_sums_host(x_host: torch.Tensor, layout: int = ROW_WISE, variant: int = AUTO,
                     out_host: torch.Tensor | None = None, device_buf: torch.Tensor | None = None,
                     stream=None) -> torch.Tensor:
    """End-to-end on host (ideally pinned) buffers: H2D, kernels, D2H pipelined
    inside the library; returns when out_host holds the result."""
    n, p = _shape_np(x_host, layout)
    dt = _dtype_code(x_host)
    if out_host is None:
        out_host = torch.empty_like(x_host)
    if device_buf is None:
        need = prefix_sums_host_bytes(n, p, dt, layout, variant)
        device_buf = torch.empty(need, dtype=torch.uint8, device="cuda")
    _check(lib().bulk_prefix_sums_host(x_host.data_ptr(), out_host.data_ptr(), n, p, dt, layout, variant,
                                       device_buf.data_ptr(), device_buf.numel(), _stream(stream)))
    return out_host


# ---------------------------------------------------------- triangulation
def _tri_shape(c: torch.Tensor, layout: int):
    if layout in (PACKED_ROW, PACKED_COLUMN):
        if c.dim() != 2:
            raise ValueError("packed weights are [p, K] (PACKED_ROW) or [K, p] (PACKED_COLUMN)")
        K, p = (c.shape[1], c.shape[0]) if layout == PACKED_ROW else (c.shape[0], c.shape[1])
        n = int(round((3 + (1 + 8 * K) ** 0.5) / 2))
        if (n - 1) * (n - 2) // 2 != K:
            raise ValueError("packed size K must be (n-1)(n-2)/2")
        return n, p
    if c.dim() != 3:
        raise ValueError("weights are [p, n, n] (ROW_WISE) or [n, n, p] (COLUMN_WISE)")
    if layout == ROW_WISE:
        p, n, n2 = c.shape
    else:
        n, n2, p = c.shape
    if n != n2:
        raise ValueError("weight matrices must be n x n")
    return n, p


def triangulation_workspace(n: int, p: int, dtype: int, layout: int, variant: int = AUTO) -> int:
    return int(lib().bulk_triangulation_workspace(n, p, dtype, layout, variant))


def triangulation_variant(n: int, p: int, dtype: int, layout: int, variant: int = AUTO) -> int:
    return int(lib().bulk_triangulation_variant(n, p, dtype, layout, variant))


def triangulation(c: torch.Tensor, layout: int = ROW_WISE, variant: int = AUTO, out: torch.Tensor | None = None,
                  workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """out[h] = M_h[1, n-1] of Algorithm OPT for every instance."""
    _need_cuda(c)
    n, p = _tri_shape(c, layout)
    dt = _dtype_code(c)
    if out is None:
        out = torch.empty(p, dtype=c.dtype, device=c.device)
    else:
        _check_out(out, c, (p,))
    need = triangulation_workspace(n, p, dt, layout, variant)
    wptr, wbytes = None, 0
    if need:
        if workspace is None:
            workspace = torch.empty(need, dtype=torch.uint8, device=c.device)
        _check_workspace(workspace, c)
        wptr, wbytes = workspace.data_ptr(), workspace.numel() * workspace.element_size()
    _check(lib().bulk_triangulation(c.data_ptr(), out.data_ptr(), n, p, dt, layout, variant, wptr, wbytes,
                                    _stream(stream, c)))
    return out


def triangulation_chords(c: torch.Tensor, layout: int = ROW_WISE, stream=None, out: torch.Tensor | None = None,
                         chords: torch.Tensor | None = None):
    """Values and the chords of an optimal triangulation (NEXT-1):
    returns (out [p], chords [p, n-3, 2] int16 vertex pairs)."""
    _need_cuda(c)
    n, p = _tri_shape(c, layout)
    dt = _dtype_code(c)
    if out is None:
        out = torch.empty(p, dtype=c.dtype, device=c.device)
    if chords is None:
        chords = torch.empty((p, max(n - 3, 0), 2), dtype=torch.int16, device=c.device)
    _check_out(out, c, (p,))
    _need_cuda(chords)
    if chords.device != c.device or chords.dtype != torch.int16 or chords.numel() != p * max(n - 3, 0) * 2:
        raise ValueError("chords must be [p, n-3, 2] int16 on the weights' device")
    _check(lib().bulk_triangulation_chords(c.data_ptr(), out.data_ptr(), chords.data_ptr() if chords.numel() else None,
                                           n, p, dt, layout, _stream(stream, c)))
    return out, chords


def _program_code(program):
    import numpy as np
    if hasattr(program, "array"):
        code, nregs = program.array(), program.nregs
    else:
        code, nregs = np.asarray(program, dtype=np.int32).reshape(-1, 4), 64
    return np.ascontiguousarray(code, dtype=np.int32), nregs


class Prepared:
    """An oblivious program validated, rewritten and uploaded once
    (bulk_program_prepare) for `msize`-word instance memories on `device`;
    execute(prepared, mem, layout) then does no host work per call and can be
    captured into a CUDA graph."""

    def __init__(self, program, msize: int, device="cuda", stream=None):
        code, self.nregs = _program_code(program)
        self.msize, self.t = int(msize), code.shape[0]
        self.buf = torch.empty(max(self.t, 1) * 16, dtype=torch.uint8, device=device)   # owned: lives with self
        h = ctypes.c_int64(0)
        _check(lib().bulk_program_prepare(code.ctypes.data, self.t, self.msize, self.nregs, self.buf.data_ptr(),
                                          self.buf.numel(), _stream(stream, self.buf), ctypes.byref(h)))
        self.handle = h.value
        # the upload is ordered on `stream` only: wait for it here (one-time setup), so the
        # program may then run on any stream -- an execute on another stream could otherwise
        # read the device program before its words arrive
        (stream if stream is not None else torch.cuda.current_stream(self.buf.device)).synchronize()

    def compile(self, dtype=torch.float32, layout: int = COLUMN_WISE) -> bool:
        """Build the straight-line kernel of this program for (dtype, layout)
        (bulk_program_compile, NVRTC for sm_100a; host-blocking, cached).  True
        when later execute() calls with that dtype and layout run it; False when
        the shape is not compiled (row-wise programs with msize > 95 whose
        addresses do not stay in 64-word windows) and the interpreter keeps
        serving them."""
        code = _DTYPES[dtype] if not isinstance(dtype, int) else dtype
        rc = lib().bulk_program_compile(self.handle, code, layout)
        if rc == -2:
            return False
        _check(rc)
        return True

    def source(self, dtype=torch.float32, layout: int = COLUMN_WISE) -> str:
        """The CUDA source compile() builds for (dtype, layout)."""
        code = _DTYPES[dtype] if not isinstance(dtype, int) else dtype
        n = ctypes.c_size_t(0)
        _check(lib().bulk_program_source(self.handle, code, layout, None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value)
        _check(lib().bulk_program_source(self.handle, code, layout, buf, n.value, ctypes.byref(n)))
        return buf.value.decode()

    def __del__(self):
        if getattr(self, "handle", 0) and _lib is not None:
            _lib.bulk_program_release(self.handle)
            self.handle = 0


def program_source(program, msize: int, dtype=torch.float32, layout: int = COLUMN_WISE) -> str:
    """The CUDA source bulk_program_compile would build for `program` on
    `msize`-word memories (bulk_program_generate: host only, no GPU needed)."""
    code, nregs = _program_code(program)
    d = _DTYPES[dtype] if not isinstance(dtype, int) else dtype
    n = ctypes.c_size_t(0)
    _check(lib().bulk_program_generate(code.ctypes.data, code.shape[0], int(msize), nregs, d, layout, None, 0,
                                       ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value)
    _check(lib().bulk_program_generate(code.ctypes.data, code.shape[0], int(msize), nregs, d, layout, buf, n.value,
                                       ctypes.byref(n)))
    return buf.value.decode()


def prepare(program, msize: int, device="cuda", stream=None) -> Prepared:
    return Prepared(program, msize, device, stream)


def execute(program, mem: torch.Tensor, layout: int = COLUMN_WISE, prog_buf: torch.Tensor | None = None,
            stream=None) -> torch.Tensor:
    """Bulk execution of an oblivious program (NEXT-3, Theorem 2) in
    place on mem ([p, msize] row-wise or [msize, p] column-wise).  `program`
    is a programs.Program, an int32 array [t, 4] (then nregs = 64) or a
    Prepared program (no per-call host work)."""
    _need_cuda(mem)
    if isinstance(program, Prepared):
        msize, p = _shape_np(mem, layout)
        _check(lib().bulk_execute_prepared(program.handle, mem.data_ptr(), msize, p, _dtype_code(mem), layout,
                                           _stream(stream, mem)))
        return mem
    code, nregs = _program_code(program)
    t = code.shape[0]
    msize, p = _shape_np(mem, layout)
    if prog_buf is None:
        prog_buf = torch.empty(max(t, 1) * 16, dtype=torch.uint8, device=mem.device)
    _check(lib().bulk_execute(code.ctypes.data, t, prog_buf.data_ptr(), prog_buf.numel(), mem.data_ptr(), msize, p,
                              _dtype_code(mem), layout, nregs, _stream(stream, mem)))
    return mem   # pageable H2D copies return once the host program is staged


def triangulation_host(c_host: torch.Tensor, layout: int = ROW_WISE, variant: int = AUTO,
                       out_host: torch.Tensor | None = None, device_buf: torch.Tensor | None = None,
                       stream=None) -> torch.Tensor:
    n, p = _tri_shape(c_host, layout)
    dt = _dtype_code(c_host)
    if out_host is None:
        out_host = torch.empty(p, dtype=c_host.dtype).pin_memory()
    if device_buf is None:
        need = triangulation_host_bytes(n, p, dt, layout, variant)
        device_buf = torch.empty(need, dtype=torch.uint8, device="cuda")
    _check(lib().bulk_triangulation_host(c_host.data_ptr(), out_host.data_ptr(), n, p, dt, layout, variant,
                                         device_buf.data_ptr(), device_buf.numel(), _stream(stream)))
    return out_host


# --------------------------------------------------------------- transpose
def transpose(x: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """[rows, cols] -> [cols, rows] (row-wise <-> column-wise arrangement)."""
    _need_cuda(x)
    if x.dim() != 2 or x.element_size() != 4:
        raise ValueError("transpose takes a 2-D tensor of 4-byte elements")
    rows, cols = x.shape
    if out is None:
        out = torch.empty((cols, rows), dtype=x.dtype, device=x.device)
    _check_out(out, x, (cols, rows))
    _check(lib().bulk_transpose(x.data_ptr(), out.data_ptr(), rows, cols, 4, _stream(stream, x)))
    return out


# ------------------------------------------------------ inputs / checksums
def generate_prefix(n: int, p: int, seed: int, dtype=torch.float32, layout: int = ROW_WISE, kind: str = "uniform",
                    h0: int = 0, device="cuda", out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    shape = (p, n) if layout == ROW_WISE else (n, p)
    if out is None:
        out = torch.empty(shape, dtype=dtype, device=device)
    _check(lib().bulk_generate_prefix(out.data_ptr(), n, p, h0, seed, _dtype_code(out), layout, KINDS[kind],
                                      _stream(stream, out)))
    return out


def generate_tri(n: int, p: int, seed: int, dtype=torch.float32, layout: int = ROW_WISE, h0: int = 0,
                 device="cuda", out: torch.Tensor | None = None, stream=None, kind: str = "chords") -> torch.Tensor:
    K = (n - 1) * (n - 2) // 2
    shape = {ROW_WISE: (p, n, n), COLUMN_WISE: (n, n, p), PACKED_ROW: (p, K), PACKED_COLUMN: (K, p)}[layout]
    if out is None:
        out = torch.empty(shape, dtype=dtype, device=device)
    _check(lib().bulk_generate_tri(out.data_ptr(), n, p, h0, seed, _dtype_code(out), layout, TR_KINDS[kind],
                                   _stream(stream, out)))
    return out


def checksum(values: torch.Tensor, layout: int = ROW_WISE, h0: int = 0, stream=None) -> torch.Tensor:
    """Device uint64 (as int64 tensor) fingerprint; see bulkgen.checksum."""
    _need_cuda(values)
    if values.dim() == 1:
        n, p = 1, values.shape[0]
        layout = ROW_WISE
    else:
        n, p = _shape_np(values, layout)
    acc = torch.zeros(1, dtype=torch.int64, device=values.device)
    _check(lib().bulk_checksum(values.data_ptr(), n, p, h0, layout, acc.data_ptr(), _stream(stream, values)))
    return acc


class Captured:
    """A fixed sequence of bulkobl calls recorded once as a CUDA graph and
    replayed: one host-side graph launch (a few microseconds) instead of ~7-9 us
    of binding and launch work per call -- the path for many small bulk
    problems whose kernels take about as long as their launches (PS-1: ~2 us).

        step = bo.Captured(lambda s: bo.prefix_sums(x, bo.ROW_WISE, out=y, stream=s))
        step.replay()            # same tensors, same shapes, new contents

    `fn(stream)` must launch on the stream it is given and touch only
    preallocated tensors (graph capture records pointers).  The library's
    launches are capturable: they take no work-queue slot under capture (their
    CTAs stride over tiles statically), so a replay may run beside eager calls
    on other streams.  The first call of fn runs eagerly on the capture stream
    to warm up lazily initialised state."""

    def __init__(self, fn, stream: torch.cuda.Stream | None = None):
        self.stream = stream if stream is not None else torch.cuda.Stream()
        with torch.cuda.stream(self.stream):
            fn(self.stream)
        self.stream.synchronize()
        self.graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(self.graph, stream=self.stream):
            fn(self.stream)

    def replay(self):
        self.graph.replay()


def launch_count() -> int:
    return int(lib().bulk_launch_count())


def version() -> str:
    return lib().bulk_version().decode()
