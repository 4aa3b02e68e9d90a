// exec.h -- host interface of the generic executor (exec.cu), used by api.cu.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

namespace bo {

// The uploaded form of a validated program: fused superinstructions, and WIN
// headers when windowed staging applies (wmax = the largest window, 0 = none).
struct ExecProgram {
    std::vector<int32_t> words;
    int wmax;
};
ExecProgram exec_device_program(const int32_t *prog, int64_t t, int64_t msize, int nregs);
size_t exec_staged_smem(int64_t msize, int nregs);
int launch_exec(const void *prog, int64_t t, void *mem, int64_t msize, int64_t p, int dtype, int layout, int nregs,
                int nzero, int wmax, cudaStream_t st);

}  // namespace bo
