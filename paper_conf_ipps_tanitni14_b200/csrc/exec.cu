// exec.cu -- generic bulk executor of oblivious programs (NEXT-3; Theorem 2,
// P:132-137): p threads each run the same straight-line program on their own
// instance memory, in the row-wise (j*msize + a) or column-wise (a*p + j)
// arrangement.  The instruction stream is read once per warp
// (uniform broadcast loads through L1), registers live in shared memory
// ([r][thread], conflict-free), and every LOAD/STORE of a warp touches one
// address group column-wise or 32 groups row-wise -- exactly the Theorem 2
// comparison.  Encoding: see include/bulkobl.h / programs.py.
#include "common.cuh"

namespace bo {

namespace ex {
enum { LOAD = 0, STORE, ADD, SUB, MIN, MAX, MOV, CONST };
constexpr int kThreads = 128;
}

template <typename T>
__device__ __forceinline__ T ex_add(T a, T b) { return add_wrap(a, b); }
__device__ __forceinline__ int32_t ex_sub(int32_t a, int32_t b) {
    return static_cast<int32_t>(static_cast<uint32_t>(a) - static_cast<uint32_t>(b));
}
__device__ __forceinline__ float ex_sub(float a, float b) { return __fsub_rn(a, b); }

template <typename T, int LAYOUT>
__global__ void __launch_bounds__(ex::kThreads)
exec_kernel(const int4 *__restrict__ prog, long long t, T *mem, long long msize, long long p, int nzero) {
    pdl_begin();
    extern __shared__ uint8_t smem_raw[];
    T *R = reinterpret_cast<T *>(smem_raw) + threadIdx.x;     // r[x] at R[x * kThreads]
    const long long j = blockIdx.x * static_cast<long long>(ex::kThreads) + threadIdx.x;
    const bool live = j < p;
    auto addr = [&](long long a) -> long long { return LAYOUT == BO_ROW_WISE ? j * msize + a : a * p + j; };
    // registers start at 0 (bulkobl.h); the host passes nzero = 0 when the program
    // writes every register before reading it (every builder in programs.py does)
    for (int x = 0; x < nzero; ++x) R[x * ex::kThreads] = T(0);
    for (long long i = 0; i < t; ++i) {
        const int4 ins = __ldg(prog + i);                      // same address for the whole warp
        const int x = ins.y, y = ins.z, z = ins.w;
        switch (ins.x) {
            case ex::LOAD: R[x * ex::kThreads] = live ? mem[addr(y)] : T(0); break;
            case ex::STORE: if (live) mem[addr(x)] = R[y * ex::kThreads]; break;
            case ex::ADD: R[x * ex::kThreads] = ex_add(R[y * ex::kThreads], R[z * ex::kThreads]); break;
            case ex::SUB: R[x * ex::kThreads] = ex_sub(R[y * ex::kThreads], R[z * ex::kThreads]); break;
            case ex::MIN: {                                     // "if r < s then s <- r"
                const T a = R[y * ex::kThreads], b = R[z * ex::kThreads];
                R[x * ex::kThreads] = b < a ? b : a;
                break;
            }
            case ex::MAX: {
                const T a = R[y * ex::kThreads], b = R[z * ex::kThreads];
                R[x * ex::kThreads] = a < b ? b : a;
                break;
            }
            case ex::MOV: R[x * ex::kThreads] = R[y * ex::kThreads]; break;
            case ex::CONST: {
                const uint32_t u = static_cast<uint32_t>(y);
                R[x * ex::kThreads] = *reinterpret_cast<const T *>(&u);
                break;
            }
            default: break;
        }
    }
}

int launch_exec(const void *prog, int64_t t, void *mem, int64_t msize, int64_t p, int dtype, int layout, int nregs,
                int nzero, cudaStream_t st) {
    const size_t smem = static_cast<size_t>(nregs) * ex::kThreads * 4;
    const unsigned grid = static_cast<unsigned>((p + ex::kThreads - 1) / ex::kThreads);
    const int4 *pg = static_cast<const int4 *>(prog);
    if (dtype == BO_F32) {
        if (layout == BO_ROW_WISE) launch(exec_kernel<float, BO_ROW_WISE>, grid, ex::kThreads, smem, st, pg, t, static_cast<float *>(mem), msize, p, nzero);
        else launch(exec_kernel<float, BO_COLUMN_WISE>, grid, ex::kThreads, smem, st, pg, t, static_cast<float *>(mem), msize, p, nzero);
    } else {
        if (layout == BO_ROW_WISE) launch(exec_kernel<int32_t, BO_ROW_WISE>, grid, ex::kThreads, smem, st, pg, t, static_cast<int32_t *>(mem), msize, p, nzero);
        else launch(exec_kernel<int32_t, BO_COLUMN_WISE>, grid, ex::kThreads, smem, st, pg, t, static_cast<int32_t *>(mem), msize, p, nzero);
    }
    return after_launch("exec_kernel");
}

}  // namespace bo
