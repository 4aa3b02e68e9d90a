// PDL and CTA placement: a kernel of G CTAs that each work ~T us (smem-heavy so
// 3 fit per SM), launched K times back to back: no PDL, PDL with the trigger at
// kernel start, PDL with the trigger at the end of each CTA, PDL with no trigger.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pdl_place pdl_place.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void heavy(float *out, long long cyc, int mode) {
    extern __shared__ float sm[];
    if (mode == 1) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (mode) asm volatile("griddepcontrol.wait;" ::: "memory");
    float s = threadIdx.x;
    const long long t0 = clock64();
    while (clock64() - t0 < cyc) { s = s * 1.0001f + 0.5f; sm[threadIdx.x] = s; }
    if (s == 1.0f) out[0] = sm[threadIdx.x ^ 1];
    if (mode == 2) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__global__ void spin(long long cyc) { const long long t0 = clock64(); while (clock64() - t0 < cyc) {} }

int main() {
    float *out; cudaMalloc(&out, 16);
    cudaStream_t st; cudaStreamCreate(&st);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaFuncSetAttribute(heavy, cudaFuncAttributeMaxDynamicSharedMemorySize, 72 * 1024);
    const int K = 50;
    for (int G : {64, 128, 148, 296, 444}) {
        for (long long cyc : {2000LL, 40000LL}) {
            for (int mode = 0; mode < 4; ++mode) {          // 0 none, 1 start, 2 end, 3 implicit
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3(G); cfg.blockDim = dim3(128); cfg.dynamicSmemBytes = 72 * 1024; cfg.stream = st;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
                at[0].val.programmaticStreamSerializationAllowed = 1;
                cfg.attrs = mode ? at : nullptr; cfg.numAttrs = mode ? 1 : 0;
                float best = 1e9;
                for (int rep = 0; rep < 3; ++rep) {
                    spin<<<1, 1, 0, st>>>(20000000LL);
                    cudaEventRecord(a, st);
                    for (int k = 0; k < K; ++k) cudaLaunchKernelEx(&cfg, heavy, out, cyc, mode == 3 ? 4 : mode);
                    cudaEventRecord(b, st);
                    cudaEventSynchronize(b);
                    float ms; cudaEventElapsedTime(&ms, a, b);
                    best = ms < best ? ms : best;
                }
                printf("G %4d work %6lld cyc mode %d: %.2f us/launch\n", G, cyc, mode, best * 1e3 / K);
            }
        }
    }
    return 0;
}
