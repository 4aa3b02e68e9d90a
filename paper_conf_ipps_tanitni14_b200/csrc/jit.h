// jit.h -- compiled oblivious programs (jit.cu), used by api.cu.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

namespace bo {

struct JitKernel {
    const void *kernel = nullptr;   // a cudaKernel_t of a context-independent library
};
// Build (or take from the process-wide cache) the straight-line kernel of a
// validated program for one dtype and arrangement.  BO_EUNSUPPORTED when the
// shape is not compiled (row-wise with msize > 95, or > 200000 instructions).
int jit_compile(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, int layout, JitKernel *out);
int launch_jit(const JitKernel &k, void *mem, int64_t p, cudaStream_t st);
// the generated CUDA source ("" when not compiled), for inspection and tests
std::string jit_source(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, int layout);

}  // namespace bo
