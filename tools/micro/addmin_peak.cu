// Measured ALU roof for the min-plus inner step ("R_addmin from a
// microbenchmark of the actual inner instruction mix"): the 4x4 register-tile
// chunk of tri_tiled.cu -- fp32 FADD2 (broadcast operand) + FMNMX3, int32
// VIADDMNMX -- run from registers with 8 independent tiles per thread, on every
// SM, timed with CUDA events.  Prints add-min/s.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o addmin_peak addmin_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void fp32_addmin(float *out, int iters, float seed) {
    float acc[16], a[4], b[4];
#pragma unroll
    for (int i = 0; i < 16; ++i) acc[i] = seed + i;
#pragma unroll
    for (int i = 0; i < 4; ++i) a[i] = seed * (i + 1), b[i] = seed * (i + 5);
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; v += 2) {      // 4 add-mins: 2 FADD2 + 2 FMNMX3
                const float2 s0 = __fadd2_rn(make_float2(a[u], a[u]), make_float2(b[v], b[v + 1]));
                const float2 s1 = __fadd2_rn(make_float2(a[(u + 1) & 3], a[(u + 1) & 3]), make_float2(b[v + 1], b[v]));
                acc[4 * u + v] = fminf(fminf(acc[4 * u + v], s0.x), s1.x);
                acc[4 * u + v + 1] = fminf(fminf(acc[4 * u + v + 1], s0.y), s1.y);
            }
#pragma unroll
        for (int i = 0; i < 4; ++i) a[i] = __int_as_float(__float_as_int(a[i]) ^ 1), b[i] = __int_as_float(__float_as_int(b[i]) ^ 2);
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += acc[i];
    if (s == 1.2345f) out[0] = s;
}

__global__ void i32_addmin(int *out, int iters, int seed) {
    int acc[16], a[4], b[4];
#pragma unroll
    for (int i = 0; i < 16; ++i) acc[i] = seed + i;
#pragma unroll
    for (int i = 0; i < 4; ++i) a[i] = seed * (i + 1), b[i] = seed * (i + 5);
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v)          // 2 add-mins per element per iteration
                acc[4 * u + v] = __viaddmin_s32(a[(u + 1) & 3], b[(v + 1) & 3], __viaddmin_s32(a[u], b[v], acc[4 * u + v]));
#pragma unroll
        for (int i = 0; i < 4; ++i) a[i] ^= 1, b[i] ^= 2;
    }
    int s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += acc[i];
    if (s == 12345) out[0] = s;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float *fo; int *io;
    cudaMalloc(&fo, 4); cudaMalloc(&io, 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int iters = 20000;
    for (int warps : {8, 16, 32}) {
        const int threads = 128, blocks = sms * warps * 32 / threads;
        for (int rep = 0; rep < 2; ++rep) {
            float ms;
            cudaEventRecord(a);
            fp32_addmin<<<blocks, threads>>>(fo, iters, 1.5f);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double fp = double(blocks) * threads * iters * 32 / (ms * 1e-3);   // 16 elems x 2 add-mins
            cudaEventRecord(a);
            i32_addmin<<<blocks, threads>>>(io, iters, 3);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double ip = double(blocks) * threads * iters * 32 / (ms * 1e-3);
            if (rep) printf("%2d warps/SM: fp32 FADD2+FMNMX3 %.2f T add-min/s, int32 VIADDMNMX %.2f T add-min/s\n", warps,
                            fp / 1e12, ip / 1e12);
        }
    }
    return 0;
}
