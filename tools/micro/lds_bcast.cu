// Microbenchmark: shared-memory wavefronts of LDS.128 under address sharing
// patterns (read with ncu: l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o lds_bcast lds_bcast.cu
#include <cstdio>
#include <cuda_runtime.h>
template <int MODE>
__global__ void k(float *out, int iters) {
    __shared__ float4 s[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) s[i] = make_float4(i, i + 1, i + 2, i + 3);
    __syncthreads();
    const int l = threadIdx.x & 31;
    int idx;
    if (MODE == 0) idx = l;                 // 32 distinct, conflict-free
    else if (MODE == 1) idx = l >> 1;       // pairs of adjacent lanes share
    else if (MODE == 2) idx = l & 7;        // the 4 phases repeat the same 8 addresses
    else if (MODE == 3) idx = 0;            // broadcast
    else if (MODE == 4) idx = (l & 1) * 8 + (l >> 2);   // pairs (l, l^2) share, spread
    else idx = l & 15;                      // halves repeat 16 addresses
    float4 acc = make_float4(0, 0, 0, 0);
    for (int it = 0; it < iters; ++it) {
        const float4 v = s[(idx + it * 32) & 1023];
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}
int main() {
    float *o;
    cudaMalloc(&o, 1 << 20);
    k<0><<<148, 128>>>(o, 1000);
    k<1><<<148, 128>>>(o, 1000);
    k<2><<<148, 128>>>(o, 1000);
    k<3><<<148, 128>>>(o, 1000);
    k<4><<<148, 128>>>(o, 1000);
    k<5><<<148, 128>>>(o, 1000);
    cudaDeviceSynchronize();
    printf("done\n");
    return 0;
}
