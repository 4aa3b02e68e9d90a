"""bulkgen -- seeded, counter-based synthetic inputs shared by tests and bench.

This module holds NONE of the method's arithmetic (no prefix sums, no
min-plus, no transpose): it only defines what the p input instances ARE, so
that the CPU oracle (oracle/) and the CUDA path (paper_conf_ipps_tanitni14_b200)
can be fed identical data.  The CUDA library implements the same generator on
the device (bulk_generate_* in include/bulkobl.h); tests check the two agree
bit for bit.

Generator:
    x   = seed*K_SEED + h*K_H + e*K_E          (mod 2^64)
    u   = mix64(x)                             (splitmix64 finaliser)
where h is the GLOBAL instance id (so a shard of ranks [h0, h1) generates the
same values whatever the GPU count) and e the element id inside an instance.

Prefix-sum inputs (paper: "float (32-bit) numbers", Sec. V):
    int32 'uniform':  (int32)(u >> 32)          full range, wraps (reading G13)
    fp32  'uniform':  (u >> 40) * 2^-24         in [0, 1)
    'ones':           1                         (closed-form pin 1..n)
    'arange':         e                         (closed-form pin e(e+1)/2)
    'smallint':       (u >> 60)                 integers 0..15 (exact in fp32)
Triangulation chord weights (dense n x n per instance, reading G6),
e = a*n + b, two kinds:
  'chords' (the configs' workload; TR_KINDS code 0):
    c[a][b] for b-a >= 2 and (a,b) != (0,n-1):
        int32: u >> 44  in [0, 2^20)            fp32: (u >> 40) * 2^-24
    every other entry (polygon sides, root side, lower triangle) = 0 (G8)
  'full' (parity stress; code 1): EVERY entry is non-zero.
    read entries b-a >= 2, INCLUDING the root side c[0][n-1] (P:199 adds it):
        int32: (u >> 32) mod (2B-1) - (B-1), B = 2^31 div (2(n-2)), signed,
               so |c| < 2^31 / (2(n-2)) (the ABI bound, reading G13)
        fp32:  (u >> 40) * 2^-23 - 1            signed, in [-1, 1)
    unread entries b-a <= 1 (sides, diagonal, lower triangle) hold poison:
        int32: (int32)(u >> 32) (full range)
        fp32:  by u >> 61: qNaN, +inf, -inf, +FLT_MAX, -FLT_MAX, sNaN, -0,
               a value in [-1, 1) -- any read of them changes the result
"""
from __future__ import annotations

import numpy as np

K_SEED = np.uint64(0x9E3779B97F4A7C15)
K_H = np.uint64(0xD1B54A32D192ED03)
K_E = np.uint64(0x8CB92BA72F3D8DD7)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)

ROW_WISE = 0     # [p][n]: b_j[i] at j*n + i
COLUMN_WISE = 1  # [n][p]: b_j[i] at i*p + j
PACKED_ROW = 2   # triangulation weights: [p][K], only b-a >= 2, row by row (NEXT-4)
PACKED_COLUMN = 3  # [K][p]


def mix64(z: np.ndarray) -> np.ndarray:
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z ^ (z >> np.uint64(30))
        z = z * M1
        z = z ^ (z >> np.uint64(27))
        z = z * M2
        z = z ^ (z >> np.uint64(31))
    return z


def u64(seed: int, h: np.ndarray, e: np.ndarray) -> np.ndarray:
    h = np.asarray(h, dtype=np.uint64)
    e = np.asarray(e, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = np.uint64(seed) * K_SEED + h * K_H + e * K_E
    return mix64(x)


def _prefix_values(u: np.ndarray, e: np.ndarray, dtype: str, kind: str) -> np.ndarray:
    if kind == "uniform":
        if dtype == "int32":
            return (u >> np.uint64(32)).astype(np.uint32).view(np.int32)
        return ((u >> np.uint64(40)).astype(np.float64) * 2.0 ** -24).astype(np.float32)
    if kind == "ones":
        return np.ones(u.shape, dtype=np.int32 if dtype == "int32" else np.float32)
    if kind == "arange":
        return np.broadcast_to(e, u.shape).astype(np.int32 if dtype == "int32" else np.float32)
    if kind == "smallint":
        return (u >> np.uint64(60)).astype(np.int32 if dtype == "int32" else np.float32)
    raise ValueError(f"unknown kind {kind!r}")


KINDS = {"uniform": 0, "ones": 1, "arange": 2, "smallint": 3}


def prefix_input(n: int, p: int, seed: int, dtype: str = "float32", layout: int = ROW_WISE,
                 kind: str = "uniform", h0: int = 0) -> np.ndarray:
    """p instances (global ids h0..h0+p-1) of n elements, in the given arrangement.

    Returns shape [p, n] for ROW_WISE, [n, p] for COLUMN_WISE (C-contiguous)."""
    h = np.arange(h0, h0 + p, dtype=np.uint64)[:, None]
    e = np.arange(n, dtype=np.uint64)[None, :]
    v = _prefix_values(u64(seed, h, e), e, dtype, kind)
    v = np.ascontiguousarray(v)
    return v if layout == ROW_WISE else np.ascontiguousarray(v.T)


def prefix_instances(n: int, ids, seed: int, dtype: str = "float32", kind: str = "uniform") -> np.ndarray:
    """Selected instances (global ids `ids`), row-wise [len(ids), n]."""
    h = np.asarray(ids, dtype=np.uint64)[:, None]
    e = np.arange(n, dtype=np.uint64)[None, :]
    return np.ascontiguousarray(_prefix_values(u64(seed, h, e), e, dtype, kind))


TR_KINDS = {"chords": 0, "full": 1}
# fp32 poison for the entries Algorithm OPT never reads ('full' kind), by u >> 61
_F32_POISON = np.array([0x7FC00000, 0x7F800000, 0xFF800000, 0x7F7FFFFF, 0xFF7FFFFF, 0x7FA00000, 0x80000000, 0],
                       dtype=np.uint32)


def tri_int32_bound(n: int) -> int:
    """B = 2^31 div (2(n-2)): 'full' int32 weights satisfy |c| <= B-1 (reading G13)."""
    return (1 << 31) // (2 * max(n - 2, 1))


def _tri_values(n: int, u: np.ndarray, dtype: str, kind: str = "chords") -> np.ndarray:
    a = np.arange(n)[:, None]
    b = np.arange(n)[None, :]
    if kind == "chords":
        mask = (b - a >= 2) & ~((a == 0) & (b == n - 1))
        if dtype == "int32":
            v = (u >> np.uint64(44)).astype(np.int32)
        else:
            v = ((u >> np.uint64(40)).astype(np.float64) * 2.0 ** -24).astype(np.float32)
        return np.where(mask, v, np.zeros((), dtype=v.dtype))
    if kind != "full":
        raise ValueError(f"unknown kind {kind!r}")
    read = np.broadcast_to(b - a >= 2, u.shape)
    if dtype == "int32":
        B = tri_int32_bound(n)
        v = ((u >> np.uint64(32)) % np.uint64(2 * B - 1)).astype(np.int64) - (B - 1)
        poison = (u >> np.uint64(32)).astype(np.uint32).view(np.int32)
        return np.where(read, v.astype(np.int32), poison)
    v = ((u >> np.uint64(40)).astype(np.float64) * 2.0 ** -23 - 1.0).astype(np.float32)
    pb = _F32_POISON[(u >> np.uint64(61)).astype(np.int64)]
    pb = np.where(pb == 0, v.view(np.uint32), pb)
    return np.where(read, v, pb.view(np.float32))


def tri_instances(n: int, ids, seed: int, dtype: str = "float32", kind: str = "chords") -> np.ndarray:
    """Chord weights of selected instances, shape [len(ids), n, n]."""
    h = np.asarray(ids, dtype=np.uint64)[:, None, None]
    e = np.arange(n * n, dtype=np.uint64).reshape(1, n, n)
    return np.ascontiguousarray(_tri_values(n, u64(seed, h, e), dtype, kind))


def packed_pairs(n: int):
    """(a, b) pairs of the packed layouts, in storage order: rows a = 0..n-3,
    b = a+2..n-1 (index k(a,b) = a(n-2) - a(a-1)/2 + (b-a-2))."""
    return [(a, b) for a in range(n - 2) for b in range(a + 2, n)]


def tri_input(n: int, p: int, seed: int, dtype: str = "float32", layout: int = ROW_WISE,
              h0: int = 0, kind: str = "chords") -> np.ndarray:
    """Chord weights: ROW_WISE [p, n, n] (c[h*n*n + a*n + b]), COLUMN_WISE
    [n, n, p] (c[(a*n + b)*p + h]), PACKED_ROW [p, K], PACKED_COLUMN [K, p]."""
    v = tri_instances(n, np.arange(h0, h0 + p), seed, dtype, kind)
    if layout == ROW_WISE:
        return v
    if layout == COLUMN_WISE:
        return np.ascontiguousarray(np.moveaxis(v, 0, 2))
    pr = packed_pairs(n)
    a = np.array([x for x, _ in pr], dtype=np.int64)
    b = np.array([y for _, y in pr], dtype=np.int64)
    pk = np.ascontiguousarray(v[:, a, b]) if len(pr) else np.zeros((p, 0), dtype=v.dtype)
    return pk if layout == PACKED_ROW else np.ascontiguousarray(pk.T)


def checksum(values: np.ndarray, layout: int = ROW_WISE, h0: int = 0) -> int:
    """Order-independent fingerprint of a bulk result:
        sum over (h, e) of mix64(bits(v)*K_SEED + h*K_H + e*K_E)  mod 2^64.
    values: [p, n] row-wise / [n, p] column-wise, or [p] per-instance results."""
    v = np.ascontiguousarray(values)
    bits = v.view(np.uint32).astype(np.uint64)
    if v.ndim == 1:
        bits = bits[:, None]
    elif layout == COLUMN_WISE:
        bits = bits.T
    p, n = bits.shape
    h = np.arange(h0, h0 + p, dtype=np.uint64)[:, None]
    e = np.arange(n, dtype=np.uint64)[None, :]
    with np.errstate(over="ignore"):
        t = mix64(bits * K_SEED + h * K_H + e * K_E)
        return int(np.sum(t, dtype=np.uint64))
