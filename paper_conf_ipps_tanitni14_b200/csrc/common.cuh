// common.cuh -- shared device/host helpers for libbulkobl (sm_100a only).
// PTX wrappers for mbarrier / TMA (cp.async.bulk.tensor) / bulk groups,
// tensor-map encoding through the driver entry point, launch bookkeeping.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdint.h>

#include <atomic>
#include <string>
#include <utility>

#include "../../include/bulkobl.h"

namespace bo {

// ---------------------------------------------------------------- errors
void set_error(const std::string &msg);
int fail(int status, const std::string &msg);
int cuda_check(cudaError_t e, const char *what);
extern std::atomic<uint64_t> g_launches;
inline void count_launch(uint64_t k = 1) { g_launches.fetch_add(k, std::memory_order_relaxed); }

// After a launch: record it and turn a launch error into BO_ECUDA.
inline int after_launch(const char *what) {
    count_launch();
    return cuda_check(cudaGetLastError(), what);
}

// Programmatic dependent launch (PDL).  Every kernel is launched with
// cudaLaunchAttributeProgrammaticStreamSerialization and begins with
// pdl_begin() = griddepcontrol.wait: it waits for the previous kernel in the
// stream to complete and its memory to be visible before it touches global
// memory, so stream order is kept, but the launch itself is processed while
// the predecessor drains (measured on B200, tools/micro/pdl_gap.cu: a 128 KB
// kernel 3.5 -> 1.2 us per launch back to back, a 16 MB one 8.2 -> 5.7 us).
// No kernel calls griddepcontrol.launch_dependents early: the implicit trigger
// at exit keeps the successor's CTAs off SMs the predecessor still occupies
// (an early trigger packed a small successor grid onto the few idle SMs:
// 1024 64-gons 17 -> 23 us; tools/micro/pdl_place.cu: the implicit trigger
// keeps ~90 % of the gain).  Without the attribute the wait is a no-op.
__device__ __forceinline__ void pdl_begin() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
template <typename... KArgs, typename... Args>
inline void launch(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args &&...args) {
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);   // errors: after_launch()
}

// Opt a kernel into `bytes` of dynamic shared memory on the current device;
// done once per (device, kernel) -- processes may drive several GPUs.
bool ensure_dyn_smem(const void *func, int bytes);

// Resident CTAs per SM of `func` at this block size and dynamic shared memory,
// memoised per (device, kernel, threads, smem): the occupancy query is a
// per-call host cost the small configs (a few microseconds of GPU time) feel.
int max_blocks_per_sm(const void *func, int threads, size_t smem);

inline int num_sms() {
    static int sms = [] {
        int dev = 0, v = 148;
        if (cudaGetDevice(&dev) == cudaSuccess)
            cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
        return v;
    }();
    return sms;
}

// ---------------------------------------------------------------- TMA host
// 2-D tensor map over a row-major [rows][cols] array of 4-byte elements.
// box = {box_cols, box_rows}; swizzle 128B requires box_cols*4 <= 128.
bool make_tmap_2d(CUtensorMap *map, const void *base, uint64_t rows, uint64_t cols,
                  uint32_t box_rows, uint32_t box_cols, CUtensorMapSwizzle swz,
                  CUtensorMapL2promotion l2 = CU_TENSOR_MAP_L2_PROMOTION_L2_256B);

inline bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// ---------------------------------------------------------------- device PTX
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// The first A-byte aligned address of a dynamic shared-memory buffer, as an
// offset from it: a pointer rebuilt from an integer loses the shared address
// space, and the compiler then emits generic LD / ST for every access (and
// cannot reorder them) -- measured in ps_fused_row_tma's scan.
template <int A>
__device__ __forceinline__ uint8_t *smem_align(uint8_t *raw) {
    return raw + ((A - (smem_u32(raw) & (A - 1))) & (A - 1));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
    uint32_t addr = smem_u32(bar);
    uint32_t done;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(addr), "r"(phase)
            : "memory");
    } while (!done);
}

// TMA: global (tensor map) -> shared, completion counted on an mbarrier.
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int c0, int c1,
                                            uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}

// TMA: shared -> global (tensor map), tracked by bulk async-groups.
__device__ __forceinline__ void tma_store_2d(const CUtensorMap *map, const void *src, int c0,
                                             int c1) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                     reinterpret_cast<uint64_t>(map)),
                 "r"(smem_u32(src)), "r"(c0), "r"(c1)
                 : "memory");
}

__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }

template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait() {
    asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}

// Order this thread's generic-proxy smem writes before later async-proxy
// (TMA) reads of the same smem.
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// ---------------------------------------------------------------- work queue
// Dynamic tile scheduler for persistent kernels: CTA b starts on tile b, then
// claims gridDim.x + (ticket) until the tiles run out, so SMs that run faster
// (L2 die, DRAM channel mix) take more tiles.  The last CTA to retire resets
// the slot, so no host memset is needed between launches.  The host gives each
// (device, stream) its own slot (work_slot_for, api.cu), and none (-1) to a
// launch being captured into a graph: with no slot the CTAs stride statically
// (tile b, b + gridDim.x, ...), so no two grids can ever share a counter.
struct WorkSlot {
    unsigned long long next;
    unsigned int done;
    unsigned int pad;
};
constexpr int kWorkSlots = 256;
int work_slot_for(cudaStream_t st);

// next tile after `cur` for this CTA: dynamic (w != nullptr) or static striding
__device__ __forceinline__ long long claim_tile(WorkSlot *w, long long cur) {
    if (w == nullptr) return cur + static_cast<long long>(gridDim.x);
    return static_cast<long long>(gridDim.x) + static_cast<long long>(atomicAdd(&w->next, 1ull));
}
__device__ __forceinline__ void retire_cta(WorkSlot *w) {
    if (w == nullptr) return;
    __threadfence();
    if (atomicAdd(&w->done, 1u) == gridDim.x - 1) {
        w->next = 0;
        w->done = 0;
        __threadfence();
    }
}

__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// Byte offset of the 16-byte chunk `chunk` (0..7) of row `row` in a tile whose
// rows are 128 B and which TMA wrote with CU_TENSOR_MAP_SWIZZLE_128B
// (tile base 1024-byte aligned): chunk' = chunk ^ (row % 8).
__device__ __forceinline__ uint32_t swz128(uint32_t row, uint32_t chunk) {
    return row * 128u + ((chunk ^ (row & 7u)) << 4);
}

// ---------------------------------------------------------------- weights
// Index of the chord weight c[a][b] of instance h in the four weight layouts
// (include/bulkobl.h): dense row-wise c[h*n*n + a*n + b], dense column-wise
// c[(a*n + b)*p + h], packed (b - a >= 2 only, K = (n-1)(n-2)/2 per instance,
// k = a(n-2) - a(a-1)/2 + (b-a-2)) row-wise c[h*K + k] or column-wise c[k*p + h].
__host__ __device__ __forceinline__ long long tri_c_index(int layout, long long h, long long n, long long p,
                                                          long long a, long long b) {
    if (layout <= BO_COLUMN_WISE) {
        const long long e = a * n + b;
        return layout == BO_ROW_WISE ? h * n * n + e : e * p + h;
    }
    const long long K = (n - 1) * (n - 2) / 2, k = a * (n - 2) - a * (a - 1) / 2 + (b - a - 2);
    return layout == BO_PACKED_ROW ? h * K + k : k * p + h;
}

// ---------------------------------------------------------------- arithmetic
// int32 adds wrap mod 2^32 (two's complement), done in uint32 to avoid UB.
__device__ __forceinline__ int32_t add_wrap(int32_t a, int32_t b) {
    return static_cast<int32_t>(static_cast<uint32_t>(a) + static_cast<uint32_t>(b));
}
__device__ __forceinline__ float add_wrap(float a, float b) { return __fadd_rn(a, b); }

}  // namespace bo
