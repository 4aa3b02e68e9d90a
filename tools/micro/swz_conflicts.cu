// Where do the shared-memory "bank conflicts" ncu reports for the TMA kernels
// (ps_fused_row_tma, transpose_tma_kernel) come from?  VERDICT r01 #8.
//
// One kernel, the access pattern of ps_fused_row_tma's scan: 128 threads, a
// ring of 8 stages of [128 rows x 128 B] (16 KB, 1024-byte aligned); thread t
// reads and writes its row's 8 16-byte chunks at the SWIZZLE_128B position
// chunk ^ (t % 8) (common.cuh swz128), one __syncthreads per stage.
//   mode 0: LSU only -- nothing else touches shared memory.
//   mode 1: the same, while the async proxy (the TMA engine, here 1-D
//           cp.async.bulk) streams 16 KB into the stage 4 ahead and 16 KB out of
//           the stage 4 behind, completing on an mbarrier / bulk group, like the
//           real kernel's loads and stores.
// If mode 0 counts ~0 conflicts and mode 1 counts many, the counter in the real
// kernels is arbitration with the TMA engine's shared-memory traffic, not a
// conflict of the swizzled 128-bit LSU accesses.  Run under ncu with
//   l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,
//   l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,
//   l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,
//   l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o swz_conflicts swz_conflicts.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kStages = 8, kBox = 16384, kThreads = 128;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ uint32_t swz128(uint32_t row, uint32_t chunk) {
    return row * 128u + ((chunk ^ (row & 7u)) << 4);
}

__global__ void __launch_bounds__(kThreads, 1) scan_ring(const uint8_t *src, uint8_t *dst, int iters, int mode) {
    extern __shared__ uint8_t raw[];
    uint8_t *buf = raw + ((1024u - (smem_u32(raw) & 1023u)) & 1023u);   // stays a shared-memory pointer
    __shared__ __align__(8) uint64_t bar[kStages];
    const int tid = threadIdx.x;
    for (int i = tid; i < kStages * kBox / 16; i += kThreads) reinterpret_cast<uint4 *>(buf)[i] = make_uint4(i, 0, 0, 0);
    if (tid == 0)
        for (int s = 0; s < kStages; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncthreads();
    const size_t blk = static_cast<size_t>(blockIdx.x) * iters;
    uint32_t phase[kStages] = {};
    float acc = 0.f;
    for (int it = 0; it < iters; ++it) {
        const int s = it % kStages;
        if (mode == 1 && tid == 0) {
            const int sl = (s + 4) % kStages, ss = (s + kStages - 4) % kStages;
            // load 16 KB into stage s+4 (async proxy writes shared memory)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[sl])), "r"(kBox) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(buf + sl * kBox)),
                         "l"(src + ((blk + it) % 4096) * kBox), "r"(kBox), "r"(smem_u32(&bar[sl]))
                         : "memory");
            // store 16 KB from stage s-4 (async proxy reads shared memory)
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + ((blk + it) % 4096) * kBox),
                         "r"(smem_u32(buf + ss * kBox)), "r"(kBox)
                         : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            asm volatile("cp.async.bulk.wait_group.read 2;" ::: "memory");
            // wait for the load issued 4 iterations ago into this stage
            if (it >= 4) {
                uint32_t ok = 0;
                while (!ok)
                    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                                 : "=r"(ok) : "r"(smem_u32(&bar[s])), "r"(phase[s]) : "memory");
                phase[s] ^= 1;
            }
        }
        __syncthreads();
        uint8_t *box = buf + s * kBox;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            uint4 *q = reinterpret_cast<uint4 *>(box + swz128(tid, k));
            uint4 v = *q;
            acc += __uint_as_float(v.x) + __uint_as_float(v.y) + __uint_as_float(v.z) + __uint_as_float(v.w);
            v.x += 1; v.y ^= 3; v.z += 2; v.w ^= 5;
            *q = v;
        }
        __syncthreads();
    }
    if (tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    if (acc == 1.2345f) dst[0] = 1;
}

int main() {
    uint8_t *src, *dst;
    cudaMalloc(&src, size_t(4096) * kBox);
    cudaMalloc(&dst, size_t(4096) * kBox);
    const int smem = kStages * kBox + 1024;
    cudaFuncSetAttribute(scan_ring, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int mode = 0; mode < 2; ++mode) {
        scan_ring<<<sms, kThreads, smem>>>(src, dst, 512, mode);
        cudaError_t e = cudaDeviceSynchronize();
        printf("mode %d (%s): %s\n", mode, mode ? "LSU + async-proxy bulk load/store" : "LSU only",
               cudaGetErrorString(e));
    }
    return 0;
}
