// Back-to-back launch cost on B200: K launches of a kernel that reads 64 KB per
// CTA-set, plain stream order vs programmatic dependent launch (PDL).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pdl_gap pdl_gap.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void work(const float4 *in, float *out, int n4, int pdl) {
    if (pdl) asm volatile("griddepcontrol.launch_dependents;");
    if (pdl) asm volatile("griddepcontrol.wait;" ::: "memory");
    float s = 0.f;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += gridDim.x * blockDim.x) {
        float4 v = in[i];
        s += v.x + v.y + v.z + v.w;
    }
    if (s == 12345.f) out[0] = s;
}

__global__ void spin(long long cyc) {
    const long long t0 = clock64();
    while (clock64() - t0 < cyc) {}
}

int main() {
    const int K = 200;
    for (size_t bytes : {size_t(0), size_t(1) << 17, size_t(1) << 24, size_t(1) << 26}) {
        const int n4 = static_cast<int>(bytes / 16);
        const int copies = bytes ? static_cast<int>(std::max<size_t>(1, (size_t(300) << 20) / bytes)) : 1;
        float4 *in; float *out;
        cudaMalloc(&in, std::max<size_t>(bytes, 16) * copies);
        cudaMalloc(&out, 16);
        cudaMemset(in, 0, std::max<size_t>(bytes, 16) * copies);
        cudaStream_t st; cudaStreamCreate(&st);
        cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
        for (int pdl = 0; pdl < 2; ++pdl) {
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(148 * 4); cfg.blockDim = dim3(256); cfg.stream = st;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[0].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = pdl ? at : nullptr; cfg.numAttrs = pdl ? 1 : 0;
            for (int rep = 0; rep < 3; ++rep) {
                spin<<<1, 1, 0, st>>>(20000000LL);   // host queues every launch meanwhile
                cudaEventRecord(a, st);
                for (int k = 0; k < K; ++k)
                    cudaLaunchKernelEx(&cfg, work, in + (size_t)(k % copies) * n4, out, n4, pdl);
                cudaEventRecord(b, st);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b);
                if (rep == 2) printf("bytes %10zu pdl %d: %.2f us/launch (%.0f GB/s)\n", bytes, pdl, ms * 1e3 / K,
                                     bytes / (ms * 1e-3 / K) / 1e9);
            }
        }
        cudaFree(in); cudaFree(out);
    }
    return 0;
}
