// tri.cu -- bulk optimal convex-polygon triangulation (Algorithm OPT,
// P:174-200; Parallel Algorithm OPT).
//
// Per instance h, with M[i,i] = 0:
//     M[i,j] = min_{k=i..j-1} (M[i,k] + M[k+1,j]) + c[i-1,j],   out[h] = M[1,n-1].
// Cell (i,j) needs only cells of smaller j-i, so ANY topological order --
// in particular the diagonal wavefront d = j-i = 1..n-2 -- gives the same
// values, and because min is exact and every sum keeps its association
// ((M[i,k] + M[k+1,j]) then + c), the k order of the min is free: results are
// bit-identical to the sequential algorithm for int32 and for finite fp32.
//
//   THREAD_REG  thread per instance, whole table in registers (fully unrolled,
//               n a template parameter, 3 <= n <= 18).
//   UMM_GLOBAL  the paper's kernel: thread per instance, M in global memory
//               in the same arrangement as c (row-wise (n-1)^2 h + ..., or
//               column-wise interleaved cell*p + h), 64-thread
//               blocks, one 32-bit access per step.
//   SMEM_WARP   warp per instance, M in shared memory (row stride SP = 1 mod
//               32 so diagonal-parallel row AND column reads are
//               bank-conflict-free), diagonal wavefront, long diagonals split
//               the k range over g lanes + xor-shuffle min.
//   TILED       (tri_tiled.cu) warp per instance, 4x4 register tiles.
#include "common.cuh"

#include <climits>

namespace bo {

template <typename T>
struct MinPlus;
template <>
struct MinPlus<int32_t> {
    __host__ __device__ static constexpr int32_t inf() { return INT32_MAX; }
    // min(a + b, s): one VIADDMNMX on sm_100a
    static __device__ __forceinline__ int32_t addmin(int32_t a, int32_t b, int32_t s) {
        return __viaddmin_s32(a, b, s);
    }
    static __device__ __forceinline__ int32_t add(int32_t a, int32_t b) { return add_wrap(a, b); }
    static __device__ __forceinline__ int32_t min(int32_t a, int32_t b) { return ::min(a, b); }
};
template <>
struct MinPlus<float> {
    __host__ __device__ static constexpr float inf() { return __builtin_huge_valf(); }
    static __device__ __forceinline__ float addmin(float a, float b, float s) {
        return fminf(__fadd_rn(a, b), s);
    }
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float min(float a, float b) { return fminf(a, b); }
};

__host__ __device__ __forceinline__ long long c_index(int layout, long long h, long long n, long long p,
                                                      long long a, long long b) {
    return tri_c_index(layout, h, n, p, a, b);
}

// -------------------------------------------------------------- THREAD_REG
#ifndef BO_REG_THREADS
#define BO_REG_THREADS 256   // measured TR-1 column-wise: 256 7.11 us, 128 7.32, 64 7.22, 32 7.22
#endif
template <typename T, int N, int LAYOUT>   // layout a template parameter: the 105+ weight
__global__ void __launch_bounds__(BO_REG_THREADS)      // loads must be branch-free so they issue early
tri_thread_reg(const T *__restrict__ c, T *__restrict__ out, long long p) {
    pdl_begin();
    constexpr int layout = LAYOUT;
    using Op = MinPlus<T>;
    const long long h = static_cast<long long>(blockIdx.x) * BO_REG_THREADS + threadIdx.x;
    if (h >= p) return;
    T M[N][N];                         // 1-based M[i][j], i <= j; all indices compile-time
#pragma unroll
    for (int i = 1; i <= N - 1; ++i) M[i][i] = T(0);
#pragma unroll
    for (int i = N - 2; i >= 1; --i) {
#pragma unroll
        for (int j = i + 1; j <= N - 1; ++j) {
            T s = Op::inf();
#pragma unroll
            for (int k = i; k <= j - 1; ++k) s = Op::addmin(M[i][k], M[k + 1][j], s);
            M[i][j] = Op::add(s, __ldg(c + c_index(layout, h, N, p, i - 1, j)));
        }
    }
    out[h] = M[1][N - 1];
}

// THREAD_REG fed by TMA: persistent CTAs of W warps sharing a ring of S batch
// slots; a batch = 32 instances (one per lane), whose weights are staged in
// shared memory by cp.async.bulk.tensor boxes of [32 instances x 32 elements]
// (row-wise c: box = 32 consecutive elements of 32 instances, 128B-swizzled,
// read back as conflict-free 128-bit chunks; column-wise c: box = 32 elements
// x 32 consecutive instances, one word per lane).  Batch i of the CTA goes to
// slot i % S and is computed by warp i % W; when a warp finishes batch i it
// issues batch i + S into the slot it just released, so S - W batches are in
// flight while W compute.  (Measured: p = 2^20 156 us with W = 2, S = 4 against
// 161 us with one-warp CTAs; p = 65536 is DRAM-bound either way, 14.4 us.)  Only elements up to the last one Algorithm OPT
// reads are fetched.
// Box width in elements of the row-wise TMA batches: 32 (128-byte rows, 128B
// swizzle), or 16 (64-byte rows, 64B swizzle) where that fetches fewer of the
// elements past the last one Algorithm OPT reads: n = 8, 48 of 64 elements
// (192 instead of 256 bytes per instance; with L2 promotion to 64 B, 8-gons at
// p = 4M 159 -> 131 us).  n = 10 (80 of 100) measured slower (76 vs 68 us at p = 2^20).
__host__ __device__ constexpr int reg_tma_box_width(int N, int layout) {
    return layout == BO_ROW_WISE && N == 8 ? 16 : 32;
}

template <typename T, int N, int LAYOUT, int S, int W>
__global__ void __launch_bounds__(32 * W)
tri_thread_reg_tma(const __grid_constant__ CUtensorMap cmap, T *__restrict__ out, long long p, long long nbatch) {
    pdl_begin();
    using Op = MinPlus<T>;
    constexpr int NE = LAYOUT == BO_PACKED_ROW ? (N - 1) * (N - 2) / 2   // packed: every weight is read
                                               : (N - 3) * N + N;        // c[N-3][N-1] is the last one read
    constexpr int BW = reg_tma_box_width(N, LAYOUT);   // elements per box row (32, or 16 with 64B swizzle)
    constexpr int NB = (NE + BW - 1) / BW;
    constexpr uint32_t kBoxBytes = 32u * BW * 4u;
    constexpr uint32_t kBatchBytes = NB * kBoxBytes;
    // slot i % S of batch i is then always one of warp i % W's own slots: a warp
    // can never wait on (or refill) a slot whose previous batch another warp
    // still holds, so one full barrier per slot and its phase parity suffice
    static_assert(S % W == 0 && S / W >= 1, "each warp owns S / W ring slots");
    extern __shared__ uint8_t smem_raw[];
    uint8_t *buf = smem_align<1024>(smem_raw);
    uint64_t *bar = reinterpret_cast<uint64_t *>(buf + S * kBatchBytes);
    const int t = threadIdx.x & 31, warp = threadIdx.x >> 5;
    auto issue = [&](long long i) {                  // batch i of this CTA -> ring slot i % S
        const long long b = blockIdx.x + i * gridDim.x;
        if (b >= nbatch) return;
        const int sl = static_cast<int>(i % S);
        uint8_t *dst = buf + sl * kBatchBytes;
        mbar_arrive_expect_tx(&bar[sl], kBatchBytes);
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            if (LAYOUT != BO_COLUMN_WISE) tma_load_2d(dst + k * kBoxBytes, &cmap, k * BW, static_cast<int>(b * 32), &bar[sl]);
            else tma_load_2d(dst + k * kBoxBytes, &cmap, static_cast<int>(b * 32), k * 32, &bar[sl]);
        }
    };
    if (threadIdx.x == 0) {
        prefetch_tmap(&cmap);
#pragma unroll
        for (int k = 0; k < S; ++k) mbar_init(&bar[k], 1);
        fence_barrier_init();
        for (int k = 0; k < S; ++k) issue(k);
    }
    if (W > 1) __syncthreads();
    else __syncwarp();
    for (long long i = warp;; i += W) {
        const long long b = blockIdx.x + i * gridDim.x;
        if (b >= nbatch) break;
        const int sl = static_cast<int>(i % S);
        mbar_wait(&bar[sl], static_cast<uint32_t>((i / S) & 1));
        const uint8_t *cur = buf + sl * kBatchBytes;
        auto cl = [&](int e) -> T {                 // e = dense index a*N + b (compile time)
            if (LAYOUT == BO_PACKED_ROW) {
                const int a = e / N, b = e % N;
                e = a * (N - 2) - a * (a - 1) / 2 + (b - a - 2);
            }
            const uint8_t *box = cur + (e / BW) * kBoxBytes;
            if (LAYOUT != BO_COLUMN_WISE) {
                // 128B swizzle: chunk ^ (row % 8) in 128-byte rows; 64B swizzle: chunk ^ ((row / 2) % 4)
                // in 64-byte rows -- either way the 8 lanes of a phase hit 8 distinct 16-byte slots
                const int ch = (e % BW) >> 2;
                const uint32_t off = BW == 32 ? swz128(t, ch) : t * 64u + ((ch ^ ((t >> 1) & 3)) << 4);
                const uint4 v = *reinterpret_cast<const uint4 *>(box + off);
                const uint32_t w = (e & 3) == 0 ? v.x : (e & 3) == 1 ? v.y : (e & 3) == 2 ? v.z : v.w;
                return *reinterpret_cast<const T *>(&w);
            }
            return *reinterpret_cast<const T *>(box + (e & 31) * 128 + t * 4);
        };
        T M[N][N];
#pragma unroll
        for (int ii = 1; ii <= N - 1; ++ii) M[ii][ii] = T(0);
#pragma unroll
        for (int ii = N - 2; ii >= 1; --ii) {
#pragma unroll
            for (int j = ii + 1; j <= N - 1; ++j) {
                T s = Op::inf();
#pragma unroll
                for (int k = ii; k <= j - 1; ++k) s = Op::addmin(M[ii][k], M[k + 1][j], s);
                M[ii][j] = Op::add(s, cl((ii - 1) * N + j));
            }
        }
        const long long h = b * 32 + t;
        if (h < p) out[h] = M[1][N - 1];
        __syncwarp();                                        // every lane is done with slot i % S
        if (t == 0) issue(i + S);
    }
}

// THREAD_REG on packed row-wise weights (NEXT-4): a batch of 32 consecutive
// instances is one contiguous run of 32*K words, moved by a single 1-D bulk
// copy (cp.async.bulk) into shared memory; thread t reads its instance's
// weights at t*K + k (K odd for every n = 0,1 mod 4... and any odd stride is
// bank-conflict-free).  Persistent CTAs, two buffers: the next batch streams
// in while the current one computes.  A ragged last batch reads global memory.
__device__ __forceinline__ void bulk_load_1d(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

template <typename T, int N>
__global__ void __launch_bounds__(32)
tri_thread_reg_packed(const T *__restrict__ c, T *__restrict__ out, long long p, long long nbatch) {
    pdl_begin();
    using Op = MinPlus<T>;
    constexpr int K = (N - 1) * (N - 2) / 2;
    constexpr uint32_t kBatchBytes = 32u * K * sizeof(T);
    extern __shared__ uint8_t smem_raw[];
    uint8_t *buf = smem_align<128>(smem_raw);
    uint64_t *bar = reinterpret_cast<uint64_t *>(buf + 2 * ((kBatchBytes + 127) & ~127u));
    const uint32_t stride = (kBatchBytes + 127) & ~127u;
    const int t = threadIdx.x;
    const long long nfull = p / 32;                      // batches that are complete
    auto issue = [&](long long i) {
        const long long b = blockIdx.x + i * gridDim.x;
        if (b >= nfull) return;
        mbar_arrive_expect_tx(&bar[i & 1], kBatchBytes);
        bulk_load_1d(buf + (i & 1) * stride, c + b * 32 * K, kBatchBytes, &bar[i & 1]);
    };
    if (t == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        fence_barrier_init();
        issue(0);
    }
    __syncwarp();
    for (long long i = 0;; ++i) {
        const long long b = blockIdx.x + i * gridDim.x;
        if (b >= nbatch) break;
        if (t == 0) issue(i + 1);
        const bool full = b < nfull;
        if (full) mbar_wait(&bar[i & 1], static_cast<uint32_t>((i >> 1) & 1));
        const T *cur = reinterpret_cast<const T *>(buf + (i & 1) * stride) + t * K;
        const long long h = b * 32 + t;
        const T *g = c + (h < p ? h : 0) * K;
        auto cl = [&](int a, int bb) -> T {
            const int k = a * (N - 2) - a * (a - 1) / 2 + (bb - a - 2);
            return full ? cur[k] : __ldg(g + k);
        };
        T M[N][N];
#pragma unroll
        for (int ii = 1; ii <= N - 1; ++ii) M[ii][ii] = T(0);
#pragma unroll
        for (int ii = N - 2; ii >= 1; --ii) {
#pragma unroll
            for (int j = ii + 1; j <= N - 1; ++j) {
                T s = Op::inf();
#pragma unroll
                for (int k = ii; k <= j - 1; ++k) s = Op::addmin(M[ii][k], M[k + 1][j], s);
                M[ii][j] = Op::add(s, cl(ii - 1, j));
            }
        }
        if (h < p) out[h] = M[1][N - 1];
        __syncwarp();
    }
}

// -------------------------------------------------------------- UMM_GLOBAL
template <typename T>
__global__ void __launch_bounds__(64)
tri_umm_global(const T *__restrict__ c, T *__restrict__ out, T *M, long long n, long long p, int layout) {
    pdl_begin();
    const long long h = blockIdx.x * 64LL + threadIdx.x;
    if (h >= p) return;
    const long long n1 = n - 1;
    auto mi = [&](long long i, long long j) -> long long {
        const long long cell = (i - 1) * n1 + (j - 1);
        return layout == BO_ROW_WISE ? h * n1 * n1 + cell : cell * p + h;
    };
    for (long long i = 1; i <= n - 1; ++i) M[mi(i, i)] = T(0);
    for (long long i = n - 2; i >= 1; --i) {
        for (long long j = i + 1; j <= n - 1; ++j) {
            T s = MinPlus<T>::inf();
            for (long long k = i; k <= j - 1; ++k) {
                const T r = MinPlus<T>::add(M[mi(i, k)], M[mi(k + 1, j)]);
                s = r < s ? r : s;
            }
            M[mi(i, j)] = MinPlus<T>::add(s, c[c_index(layout, h, n, p, i - 1, j)]);
        }
    }
    out[h] = M[mi(1, n - 1)];
}

// --------------------------------------------------------------- SMEM_WARP
// Table S (0-based a = i-1, b = j-1), row stride SP: S[a*SP + b] = M[a+1][b+1]
// for b >= a; before cell (a,b) is computed it holds c[a][b+1].
template <typename T>
__global__ void __launch_bounds__(512)
tri_smem_warp(const T *__restrict__ c, T *__restrict__ out, int n, long long p, int layout, int SP, int W) {
    pdl_begin();
    using Op = MinPlus<T>;
    extern __shared__ uint8_t smem_raw[];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int n1 = n - 1;
    T *S = reinterpret_cast<T *>(smem_raw) + static_cast<size_t>(warp) * n1 * SP;
    const int cells = n1 * n1;

    for (long long hb = static_cast<long long>(blockIdx.x) * W; hb < p; hb += static_cast<long long>(gridDim.x) * W) {
        const long long h = hb + warp;
        if (layout != BO_COLUMN_WISE) {
            if (h < p) {
                for (int a = 0; a < n1; ++a)
                    for (int b = a + lane; b < n1; b += 32)
                        S[a * SP + b] = b == a ? T(0) : __ldg(c + c_index(layout, h, n, p, a, b + 1));
            }
        } else {
            // column-wise c[(a*n+b)*p + h]: consecutive threads take consecutive
            // instances of the CTA so every 32-byte sector is fully used.
            __syncthreads();
            T *S0 = reinterpret_cast<T *>(smem_raw);
            for (int f = tid; f < W * cells; f += blockDim.x) {
                const int w = f % W, cell = f / W;
                const int a = cell / n1, b = cell % n1;
                if (b < a || hb + w >= p) continue;
                S0[static_cast<size_t>(w) * n1 * SP + a * SP + b] =
                    b == a ? T(0) : __ldg(c + (static_cast<long long>(a) * n + b + 1) * p + hb + w);
            }
            __syncthreads();
        }
        __syncwarp();
        if (h < p) {
            for (int d = 1; d <= n - 2; ++d) {
                const int C = n1 - d;                     // cells (a, a+d), a = 0..C-1
                int g = 1;
                while (g < 32 && C * g * 2 <= 32) g <<= 1;   // k split factor
                const int per = 32 / g;
                for (int cb = 0; cb < C; cb += per) {
                    const int a = cb + lane / g, q = lane % g;
                    const int b = a + d;
                    T s = Op::inf();
                    if (a < C) {
                        const T *row = S + a * SP;
                        for (int k = a + q; k <= b - 1; k += g) s = Op::addmin(row[k], S[(k + 1) * SP + b], s);
                    }
                    for (int off = 1; off < g; off <<= 1) s = Op::min(s, __shfl_xor_sync(0xffffffffu, s, off));
                    if (a < C && q == 0) S[a * SP + b] = Op::add(s, S[a * SP + b]);
                }
                __syncwarp();
            }
            if (lane == 0) out[h] = S[n - 2];
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------------- host
int tiled_supported(int64_t n);
size_t tiled_global_workspace(int64_t n, int64_t p);
int launch_tri_tiled_global(const void *c, void *out, void *ws, int64_t n, int64_t p, int dtype, int layout,
                            cudaStream_t st);
int launch_tri_tiled(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout, int lpi,
                     cudaStream_t st);
size_t tiled_global8_workspace(int64_t n, int64_t p);
int launch_tri_global8(const void *c, void *out, void *ws, int64_t n, int64_t p, int dtype, int layout,
                       cudaStream_t st);

static int smem_sp(int64_t n) {
    const int n1 = static_cast<int>(n - 1);
    return ((n1 - 1 + 31) / 32) * 32 + 1;   // >= n1, == 1 mod 32
}

static size_t smem_per_instance(int64_t n) { return static_cast<size_t>(n - 1) * smem_sp(n) * 4; }

int resolve_tri_variant(int64_t n, int64_t p, int dtype, int layout, int variant) {
    (void)p; (void)dtype; (void)layout;
    if (variant != BO_AUTO) return variant;
    if (n <= 16) return BO_TRI_THREAD_REG;
    // 8 lanes per instance (two tiles per lane on the long tile-diagonals) up to
    // n = 56 (1.1-1.6x faster than 16 lanes, tools/tri_time.py --cmp); 16 lanes above
    if (tiled_supported(n)) return n <= 56 ? BO_TRI_TILED_QUARTER : BO_TRI_TILED_HALF;
    return n >= 512 ? BO_TRI_TILED_GLOBAL8 : BO_TRI_TILED_GLOBAL;   // 8x8 tiles pay from n ~ 450 (tri_global8.cu)
}

size_t tri_workspace(int64_t n, int64_t p, int variant) {
    if (variant == BO_TRI_UMM_GLOBAL) return static_cast<size_t>(n - 1) * (n - 1) * p * 4;
    if (variant == BO_TRI_TILED_GLOBAL) return tiled_global_workspace(n, p);
    if (variant == BO_TRI_TILED_GLOBAL8) return tiled_global8_workspace(n, p);
    return 0;
}

// ring geometry of the TMA-fed THREAD_REG kernel: W warps per CTA (one CTA per
// SM), S batch slots of NB boxes of [32 instances x BW elements]
#ifndef BO_REG_TMA_STAGES
#define BO_REG_TMA_STAGES 4
#endif
#ifndef BO_REG_TMA_WARPS
#define BO_REG_TMA_WARPS 2
#endif
template <typename T, int N, int LAYOUT>
static int launch_reg_tma(const void *c, void *out, int64_t p, cudaStream_t st) {
    constexpr int S = BO_REG_TMA_STAGES, W = BO_REG_TMA_WARPS;
    constexpr int NE = (N - 3) * N + N;
    constexpr int BW = reg_tma_box_width(N, LAYOUT);
    constexpr int NB = (NE + BW - 1) / BW;
    constexpr size_t smem = 1024 + S * NB * (32 * BW * 4) + 8 * S;
    CUtensorMap map;
    constexpr int K = (N - 1) * (N - 2) / 2;
    // Boxes that stop short of an instance's last bytes save DRAM traffic only if L2
    // does not promote the requests back to whole 256-byte lines.  Measured: n = 8
    // (16-element boxes) p = 4M 131 us with 64B promotion, 159 us with 256B, 161 us
    // with none; n = 16 (32-element boxes, 896 of 1024 bytes) p = 65536 10.9-11.0 us
    // with 64B / 128B / none against 12.0 us with 256B (p = 2^20: 138 vs 154 us).
#ifndef BO_REG_BW16_L2
#define BO_REG_BW16_L2 CU_TENSOR_MAP_L2_PROMOTION_L2_64B
#endif
#ifndef BO_REG_L2
#define BO_REG_L2 CU_TENSOR_MAP_L2_PROMOTION_L2_64B
#endif
    const bool ok = LAYOUT == BO_ROW_WISE     ? (BW == 16 ? make_tmap_2d(&map, c, p, N * N, 32, BW, CU_TENSOR_MAP_SWIZZLE_64B,
                                                                         BO_REG_BW16_L2)
                                                          : make_tmap_2d(&map, c, p, N * N, 32, BW, CU_TENSOR_MAP_SWIZZLE_128B,
                                                                         BO_REG_L2))
                    : LAYOUT == BO_PACKED_ROW ? make_tmap_2d(&map, c, p, K, 32, 32, CU_TENSOR_MAP_SWIZZLE_128B)
                                              : make_tmap_2d(&map, c, N * N, p, 32, 32, CU_TENSOR_MAP_SWIZZLE_NONE);
    if (!ok) return fail(BO_ECUDA, "triangulation THREAD_REG: cuTensorMapEncodeTiled failed");
    auto kern = tri_thread_reg_tma<T, N, LAYOUT, S, W>;
    const bool attr = ensure_dyn_smem(reinterpret_cast<const void *>(kern), static_cast<int>(smem));
    if (!attr) return fail(BO_ECUDA, "triangulation THREAD_REG: cannot set dynamic smem");
    const long long nbatch = (p + 31) / 32;
    int per_sm = 1;
    per_sm = max_blocks_per_sm(reinterpret_cast<const void *>(kern), 32 * W, smem);
    // enough CTAs that every warp of every resident CTA has a batch
    const long long grid = std::min<long long>((nbatch + W - 1) / W, static_cast<long long>(std::max(per_sm, 1)) * num_sms());
    launch(kern, static_cast<unsigned>(grid), 32 * W, smem, st, map, static_cast<T *>(out), p, nbatch);
    return after_launch("tri_thread_reg_tma");
}

template <typename T, int N>
static int launch_reg_packed(const void *c, void *out, int64_t p, cudaStream_t st) {
    constexpr int K = (N - 1) * (N - 2) / 2;
    constexpr size_t batch = (32u * K * sizeof(T) + 127) & ~size_t(127);
    constexpr size_t smem = 128 + 2 * batch + 16;
    const bool attr = ensure_dyn_smem(reinterpret_cast<const void *>(&tri_thread_reg_packed<T, N>), static_cast<int>(smem));
    if (!attr) return fail(BO_ECUDA, "triangulation THREAD_REG packed: cannot set dynamic smem");
    const long long nbatch = (p + 31) / 32;
    int per_sm = 1;
    per_sm = max_blocks_per_sm(reinterpret_cast<const void *>(&tri_thread_reg_packed<T, N>), 32, smem);
    const long long grid = std::min<long long>(nbatch, static_cast<long long>(std::max(per_sm, 1)) * num_sms());
    launch(tri_thread_reg_packed<T, N>, static_cast<unsigned>(grid), 32, smem, st, 
        static_cast<const T *>(c), static_cast<T *>(out), p, nbatch);
    return after_launch("tri_thread_reg_packed");
}

template <typename T, int N>
static int launch_reg_n(const void *c, void *out, int64_t p, int layout, cudaStream_t st) {
    if (layout == BO_PACKED_ROW && N >= 4 && aligned16(c)) return launch_reg_packed<T, N>(c, out, p, st);
    if (p >= 32 && N >= 6 && p < (int64_t(1) << 31) && aligned16(c)) {
        if (layout == BO_ROW_WISE && (N * N) % 4 == 0) return launch_reg_tma<T, N, BO_ROW_WISE>(c, out, p, st);
        // column-wise c is already coalesced for thread-per-instance: direct loads win (measured 14.5 vs 19.3 us)
    }
    const unsigned grid = static_cast<unsigned>((p + BO_REG_THREADS - 1) / BO_REG_THREADS);
    const T *cc = static_cast<const T *>(c);
    T *oo = static_cast<T *>(out);
    switch (layout) {
        case BO_ROW_WISE: launch(tri_thread_reg<T, N, BO_ROW_WISE>, grid, BO_REG_THREADS, 0, st, cc, oo, p); break;
        case BO_COLUMN_WISE: launch(tri_thread_reg<T, N, BO_COLUMN_WISE>, grid, BO_REG_THREADS, 0, st, cc, oo, p); break;
        case BO_PACKED_ROW: launch(tri_thread_reg<T, N, BO_PACKED_ROW>, grid, BO_REG_THREADS, 0, st, cc, oo, p); break;
        default: launch(tri_thread_reg<T, N, BO_PACKED_COLUMN>, grid, BO_REG_THREADS, 0, st, cc, oo, p); break;
    }
    return after_launch("tri_thread_reg");
}

template <typename T>
static int launch_reg(const void *c, void *out, int64_t n, int64_t p, int layout, cudaStream_t st) {
    switch (n) {
#define BO_REG_CASE(N) \
    case N: return launch_reg_n<T, N>(c, out, p, layout, st);
        BO_REG_CASE(3) BO_REG_CASE(4) BO_REG_CASE(5) BO_REG_CASE(6) BO_REG_CASE(7) BO_REG_CASE(8)
        BO_REG_CASE(9) BO_REG_CASE(10) BO_REG_CASE(11) BO_REG_CASE(12) BO_REG_CASE(13) BO_REG_CASE(14)
        BO_REG_CASE(15) BO_REG_CASE(16) BO_REG_CASE(17) BO_REG_CASE(18)
#undef BO_REG_CASE
        default:
            return fail(BO_EUNSUPPORTED, "triangulation THREAD_REG supports 3 <= n <= 18");
    }
}

template <typename T>
static int launch_smem_warp(const void *c, void *out, int64_t n, int64_t p, int layout, cudaStream_t st) {
    const size_t per = smem_per_instance(n);
    if (per > 200 * 1024) return fail(BO_EUNSUPPORTED, "triangulation SMEM_WARP: table does not fit in smem");
    const bool attr = ensure_dyn_smem(reinterpret_cast<const void *>(&tri_smem_warp<T>), 227 * 1024);
    if (!attr) return fail(BO_ECUDA, "triangulation SMEM_WARP: cannot set dynamic smem");
    // warps per CTA: as many instances as fit in one SM's smem, at most 16
    int W = static_cast<int>(std::min<size_t>(16, (227 * 1024) / per));
    W = std::max(W, 1);
    const size_t smem = W * per;
    int per_sm = 1;
    per_sm = max_blocks_per_sm(reinterpret_cast<const void *>(&tri_smem_warp<T>), W * 32, smem);
    per_sm = std::max(per_sm, 1);
    const long long blocks = std::min<long long>((p + W - 1) / W, static_cast<long long>(per_sm) * num_sms() * 8);
    launch(tri_smem_warp<T>, static_cast<unsigned>(blocks), W * 32, smem, st, 
        static_cast<const T *>(c), static_cast<T *>(out), static_cast<int>(n), p, layout, smem_sp(n), W);
    return after_launch("tri_smem_warp");
}

template <typename T>
static int run_tri(const void *c, void *out, int64_t n, int64_t p, int layout, int variant, void *ws,
                   cudaStream_t st) {
    switch (variant) {
        case BO_TRI_THREAD_REG:
            return launch_reg<T>(c, out, n, p, layout, st);
        case BO_TRI_UMM_GLOBAL: {
            const unsigned grid = static_cast<unsigned>((p + 63) / 64);
            launch(tri_umm_global<T>, grid, 64, 0, st, static_cast<const T *>(c), static_cast<T *>(out),
                                                   static_cast<T *>(ws), n, p, layout);
            return after_launch("tri_umm_global");
        }
        case BO_TRI_SMEM_WARP:
            return launch_smem_warp<T>(c, out, n, p, layout, st);
        case BO_TRI_TILED:
        case BO_TRI_TILED_HALF:
        case BO_TRI_TILED_QUARTER:
            if (!tiled_supported(n)) return fail(BO_EUNSUPPORTED, "triangulation TILED supports 3 <= n <= 64");
            return launch_tri_tiled(c, out, n, p, std::is_same<T, float>::value ? BO_F32 : BO_I32, layout,
                                    variant == BO_TRI_TILED ? 32 : variant == BO_TRI_TILED_HALF ? 16 : 8, st);
        case BO_TRI_TILED_GLOBAL:
            return launch_tri_tiled_global(c, out, ws, n, p, std::is_same<T, float>::value ? BO_F32 : BO_I32, layout,
                                           st);
        case BO_TRI_TILED_GLOBAL8:
            return launch_tri_global8(c, out, ws, n, p, std::is_same<T, float>::value ? BO_F32 : BO_I32, layout, st);
        default:
            return fail(BO_EINVAL, "triangulation: unknown variant");
    }
}

int tri_dispatch(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout, int variant, void *ws,
                 cudaStream_t st) {
    if (dtype == BO_I32) return run_tri<int32_t>(c, out, n, p, layout, variant, ws, st);
    return run_tri<float>(c, out, n, p, layout, variant, ws, st);
}

}  // namespace bo
