// Measured ALU roof for the min-plus inner step ("R_addmin from a
// microbenchmark of the actual inner instruction mix"): the 4x4 register-tile
// chunk of tri_tiled.cu -- fp32 FADD2 (broadcast operand) + FMNMX3, int32
// VIADDMNMX -- run from registers on every SM, timed with CUDA events.
//
// Round 2: the loop body carries NO bookkeeping instructions.  The B operand of
// sub-step r is row r of the accumulator tile itself (so the adds cannot be
// hoisted out of the loop), which is pure register naming once the 4 sub-steps
// are unrolled; the loop is unrolled 4x more, so the only non-min-plus
// instructions are one IADD/ISETP/BRA per 512 add-mins per thread.  (The
// round-1 version varied its operands with 7 LOP3 per 32 add-mins on the same
// ALU pipe as FMNMX3 and under-stated the fp32 roof.)  Check with
//   cuobjdump -sass addmin_peak | grep -c FMNMX3   (and LOP3, FADD2, VIADDMNMX)
// and under ncu: sm__inst_executed_pipe_alu, sm__pipe_alu_cycles_active,
// sm__pipe_fma_cycles_active, sm__instruction_throughput (issue active).
// Prints add-min/s and add-min per SM per clock.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o addmin_peak addmin_peak.cu
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>

__device__ __forceinline__ float2 bcast_add(float a, float x, float y) {
    return __fadd2_rn(make_float2(a, a), make_float2(x, y));
}

// 32 add-mins: acc[u][v] = min(acc[u][v], a0[u] + acc[r][v], a1[u] + acc[r'][v])
// = 16 FADD2 + 16 FMNMX3, no other instruction
#define FP32_SUBSTEP(r, r2)                                                                      \
    _Pragma("unroll") for (int u = 0; u < 4; ++u) {                                              \
        _Pragma("unroll") for (int v = 0; v < 4; v += 2) {                                       \
            const float2 s0 = bcast_add(a0[u], acc[r][v], acc[r][v + 1]);                        \
            const float2 s1 = bcast_add(a1[u], acc[r2][v], acc[r2][v + 1]);                      \
            nxt[u][v] = fminf(fminf(acc[u][v], s0.x), s1.x);                                     \
            nxt[u][v + 1] = fminf(fminf(acc[u][v + 1], s0.y), s1.y);                             \
        }                                                                                        \
    }                                                                                            \
    _Pragma("unroll") for (int u = 0; u < 4; ++u) _Pragma("unroll") for (int v = 0; v < 4; ++v) \
        acc[u][v] = nxt[u][v];

__global__ void __launch_bounds__(128) fp32_addmin(float *out, int iters, float seed) {
    float acc[4][4], nxt[4][4], a0[4], a1[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        a0[u] = seed * (u + 1);
        a1[u] = seed * (u + 5);
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = seed + 4 * u + v + threadIdx.x;
    }
#pragma unroll 1
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            FP32_SUBSTEP(0, 1)
            FP32_SUBSTEP(1, 2)
            FP32_SUBSTEP(2, 3)
            FP32_SUBSTEP(3, 0)
        }
    }
    float s = 0;
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) s += acc[u][v];
    if (s == 1.2345f) out[0] = s;
}

// int32, two forms; the roof is the faster one.
// (a) i32_addmin: written like the fp32 kernel (operands = accumulator rows, no
//     bookkeeping).  ptxas re-associates min(min(acc, a0+x), a1+y) into its own
//     mix -- per 512 add-mins 128 VIADDMNMX + 128 VIMNMX3 + 128 VIMNMX + ~380
//     IMAD (adds on the FMA pipe, mins on the ALU pipe).
// (b) i32_addmin_xor: the round-1 form, operands varied by an XOR per iteration.
#define I32_SUBSTEP(r, r2)                                                                        \
    _Pragma("unroll") for (int u = 0; u < 4; ++u) _Pragma("unroll") for (int v = 0; v < 4; ++v)   \
        nxt[u][v] = __viaddmin_s32(a1[u], acc[r2][v], __viaddmin_s32(a0[u], acc[r][v], acc[u][v])); \
    _Pragma("unroll") for (int u = 0; u < 4; ++u) _Pragma("unroll") for (int v = 0; v < 4; ++v)   \
        acc[u][v] = nxt[u][v];

__global__ void __launch_bounds__(128) i32_addmin(int *out, int iters, int seed) {
    int acc[4][4], nxt[4][4], a0[4], a1[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        a0[u] = seed * (u + 1);
        a1[u] = seed * (u + 5);
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = seed + 4 * u + v + threadIdx.x;
    }
#pragma unroll 1
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            I32_SUBSTEP(0, 1)
            I32_SUBSTEP(1, 2)
            I32_SUBSTEP(2, 3)
            I32_SUBSTEP(3, 0)
        }
    }
    int s = 0;
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) s += acc[u][v];
    if (s == 12345) out[0] = s;
}

__global__ void __launch_bounds__(128) i32_addmin_xor(int *out, int iters, int seed) {
    int acc[16], a[4], b[4];
#pragma unroll
    for (int i = 0; i < 16; ++i) acc[i] = seed + i + threadIdx.x;
#pragma unroll
    for (int i = 0; i < 4; ++i) a[i] = seed * (i + 1), b[i] = seed * (i + 5);
    for (int it = 0; it < iters * 16; ++it) {
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


// Single-pipe probes: what each half of the fp32 mix reaches on its own pipe
// (FADD2 -> FMA pipe, FMNMX3 -> ALU pipe), 16 independent chains per thread.
// If each alone runs its pipe at ~100 %, the mix's ceiling is the dual-pipe one:
// one FADD2 (2 adds) + one FMNMX3 (2 mins) per lane per 2 cycles per SMSP =
// 128 add-mins per SM per clock; the mix kernel above shows how close the
// kernel's own instruction pairing gets.
__global__ void __launch_bounds__(128) fp32_fadd2_only(float *out, int iters, float seed) {
    float2 x[16];
    const float2 k = make_float2(seed, seed * 0.5f);
#pragma unroll
    for (int i = 0; i < 16; ++i) x[i] = make_float2(seed + i + threadIdx.x, seed - i);
#pragma unroll 1
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 16; ++r)
#pragma unroll
            for (int i = 0; i < 16; ++i) x[i] = __fadd2_rn(x[i], k);
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += x[i].x + x[i].y;
    if (s == 1.2345f) out[0] = s;
}
__global__ void __launch_bounds__(128) fp32_fmnmx3_only(float *out, int iters, float seed) {
    float x[16], y[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) x[i] = seed + i + threadIdx.x, y[i] = seed * i;
#pragma unroll 1
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 16; ++r)
#pragma unroll
            for (int i = 0; i < 16; ++i) {
                // x[i] = min(x[i], y[i], y[i+1]); y[i] = max(...) keeps the values moving
                x[i] = fminf(fminf(x[i], y[i]), y[(i + 1) & 15]);
                if (i == 15) {
#pragma unroll
                    for (int j = 0; j < 16; ++j) y[j] = x[(j + r) & 15];
                }
            }
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += x[i];
    if (s == 1.2345f) out[0] = s;
}

int main(int argc, char **argv) {
    const bool once = argc > 1 && !strcmp(argv[1], "--once");     // one launch of each (for ncu)
    int sms = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    float *fo; int *io;
    cudaMalloc(&fo, 4); cudaMalloc(&io, 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int iters = once ? 2000 : 8000;
    const double per_thread = double(iters) * 16 * 32;               // 16 sub-steps x 32 add-mins
    for (int warps : {8, 16, 32}) {
        if (once && warps != 32) continue;
        const int threads = 128, blocks = sms * warps * 32 / threads;
        for (int rep = 0; rep < (once ? 1 : 3); ++rep) {
            float ms;
            cudaEventRecord(a);
            fp32_addmin<<<blocks, threads>>>(fo, iters, 1.5f);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double fp = double(blocks) * threads * per_thread / (ms * 1e-3);
            cudaEventRecord(a);
            i32_addmin<<<blocks, threads>>>(io, iters, 3);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double ip = double(blocks) * threads * per_thread / (ms * 1e-3);
            cudaEventRecord(a);
            i32_addmin_xor<<<blocks, threads>>>(io, iters, 3);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double ix = double(blocks) * threads * per_thread / (ms * 1e-3);
            cudaEventRecord(a);
            fp32_fadd2_only<<<blocks, threads>>>(fo, iters, 1.5f);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double fa = double(blocks) * threads * double(iters) * 256 * 2 / (ms * 1e-3);   // adds/s
            cudaEventRecord(a);
            fp32_fmnmx3_only<<<blocks, threads>>>(fo, iters, 1.5f);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            const double fm = double(blocks) * threads * double(iters) * 256 * 2 / (ms * 1e-3);   // mins/s
            const double clk = clk_khz * 1e3;                         // max SM clock
            if (rep == (once ? 0 : 2))
                printf("%2d warps/SM: FADD2 alone %.2f T add/s (%.1f /SM/clk), FMNMX3 alone %.2f T min/s (%.1f /SM/clk)\n",
                       warps, fa / 1e12, fa / sms / clk, fm / 1e12, fm / sms / clk);
            if (rep == (once ? 0 : 2))
                printf("%2d warps/SM: fp32 FADD2+FMNMX3 %.2f T add-min/s (%.1f /SM/clk at max clock), "
                       "int32 (a) %.2f T add-min/s (%.1f /SM/clk), int32 (b) xor %.2f T add-min/s (%.1f /SM/clk)\n",
                       warps, fp / 1e12, fp / sms / clk, ip / 1e12, ip / sms / clk, ix / 1e12, ix / sms / clk);
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
    return 0;
}
