"""CPU checks of the program compiler's code generator (jit.cu, NEXT-3):
bulk_program_generate emits the CUDA source bulk_program_compile would build;
here that source is compiled as host C++ (IEEE binary32 arithmetic, the same
statements) and run thread by thread, and its memories must equal the oracle
interpreter's bit for bit.  The column-wise shapes (registers, and the
streaming shape with its hoisted loads and store-to-load forwarding) have no
barriers, so every thread runs on its own; the row-wise shapes are checked on
the GPU (tests/test_gpu_exec.py).  No GPU is needed."""
import os
import re
import shutil
import subprocess
import tempfile

import numpy as np
import pytest
import torch

import bulkgen
import oracle
import paper_conf_ipps_tanitni14_b200 as bo
from paper_conf_ipps_tanitni14_b200 import programs

HOST_PRELUDE = r"""
#include <cstdio>
#include <cstring>
#include <cstdint>
#include <cstdlib>
#define __global__
#define __restrict__
#define __launch_bounds__(a, b)
struct Idx { long long x; };
static Idx blockIdx, threadIdx;
static float __fadd_rn(float a, float b) { volatile float r = a + b; return r; }
static float __fsub_rn(float a, float b) { volatile float r = a - b; return r; }
static float __int_as_float(int x) { float f; std::memcpy(&f, &x, 4); return f; }
"""
HOST_MAIN = r"""
int main(int argc, char **argv) {
    long long p = atoll(argv[1]), words = atoll(argv[2]);
    T *m = new T[p * words];
    FILE *f = fopen(argv[3], "rb"); if (fread(m, sizeof(T), p * words, f) != (size_t)(p * words)) return 2; fclose(f);
    for (long long j = 0; j < p; ++j) { blockIdx.x = j / 128; threadIdx.x = j % 128; bo_prog(m, p, 0); }
    f = fopen(argv[4], "wb"); fwrite(m, sizeof(T), p * words, f); fclose(f);
    return 0;
}
"""


def _host_source(src: str) -> str:
    src = src.replace('extern "C" ', "static ")
    src = src.replace('asm volatile("griddepcontrol.wait;" ::: "memory");', "")
    src = re.sub(r"#define LDG.*\n", "#define LDG(v, a) (v) = *(const T *)((const char *)b + (a) * ps)\n", src)
    src = re.sub(r"#define STG.*\n", "#define STG(a, v) *(T *)((char *)b + (a) * ps) = (v)\n", src)
    typedef = re.search(r"typedef .* T;\n", src).group(0)
    return HOST_PRELUDE + typedef + src.replace(typedef, "") + HOST_MAIN


def _random_program(msize, nregs, t, seed, dt):
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


CASES = [("random", 8, 400, 1), ("random", 100, 800, 2), ("random", 300, 800, 3), ("bitonic", 16, 0, 0),
         ("prefix", 200, 0, 0), ("opt", 0, 0, 9)]


@pytest.mark.skipif(shutil.which("g++") is None, reason="needs g++")
@pytest.mark.parametrize("dt", ["int32", "float32"])
@pytest.mark.parametrize("kind,msize,t,seed", CASES)
def test_generated_column_source_matches_oracle(dt, kind, msize, t, seed):
    if kind == "random":
        prog = _random_program(msize, 7, t, seed, dt)
    elif kind == "bitonic":
        prog = programs.bitonic_sort(msize).array()
    elif kind == "prefix":
        prog = programs.prefix_sums(msize, dt).array()
    else:
        P = programs.optimal_triangulation(seed, dt)
        prog, msize = P.array(), P.msize
    src = bo.program_source(prog, msize, getattr(torch, dt), bo.COLUMN_WISE)
    assert ("LDG(" in src) == (msize > 128)                  # streaming shape above 128 words
    p = 37
    x = bulkgen.prefix_input(msize, p, seed=seed + 7, dtype=dt, layout=bo.COLUMN_WISE)
    if dt == "float32":
        x = (x * 8).astype(np.float32)
    ref = oracle.bulk_execute(prog, x, bo.COLUMN_WISE)
    with tempfile.TemporaryDirectory() as d:
        cpp, exe = os.path.join(d, "k.cpp"), os.path.join(d, "k")
        with open(cpp, "w") as f:
            f.write(_host_source(src))
        subprocess.run(["g++", "-O1", "-ffp-contract=off", "-fno-fast-math", "-o", exe, cpp], check=True,
                       capture_output=True)
        np.ascontiguousarray(x).tofile(os.path.join(d, "in.bin"))
        subprocess.run([exe, str(p), str(msize), os.path.join(d, "in.bin"), os.path.join(d, "out.bin")], check=True)
        got = np.fromfile(os.path.join(d, "out.bin"), dtype=x.dtype).reshape(x.shape)
    if dt == "float32":
        nan = np.isnan(ref)
        assert np.array_equal(np.isnan(got), nan)
        got, ref = got[~nan], ref[~nan]
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), (kind, msize)


def test_generate_rejects_bad_programs_and_unsupported_shapes():
    with pytest.raises(bo.BulkError):
        bo.program_source(np.array([[0, 0, 9, 0]], dtype=np.int32), 8)      # address 9 >= msize 8
    scattered = _random_program(400, 7, 500, 4, "int32")                      # row-wise, no window reuse
    with pytest.raises(bo.BulkError) as e:
        bo.program_source(scattered, 400, torch.int32, bo.ROW_WISE)
    assert e.value.status == -2
    assert "sr[" in bo.program_source(programs.prefix_sums(300), 300, torch.float32, bo.ROW_WISE)   # windowed
