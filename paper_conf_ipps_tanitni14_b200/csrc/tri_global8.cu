// tri_global8.cu -- TILED_GLOBAL8 (NEXT-2: large polygons, e.g. the paper's
// 512-gons): Algorithm OPT for one instance per CTA, with
// 8x8 register tiles over a table of 8-wide chunk-columns kept in a per-CTA
// global workspace slot (grid = #SMs, so the 148 slots -- 532 KB each at
// n = 512 -- stay L2-resident).
//
// Same vertex-coordinate reading as tri_tiled.cu (R1): X[a][a+1] = 0,
//   X[a][b] = min_{a<k<b} (X[a][k] + X[k][b]) + c[a][b],  out = X[0][n-1],
// the sums Algorithm OPT forms, each min taken over the same terms (min is
// exact, so the order is free): bit-identical to the sequential algorithm.
//
// Why 8x8 and 8-wide rows: the 4x4 kernel (TILED_GLOBAL) reads its operands
// as 16-byte pieces of 64-byte rows scattered over the table, and ncu shows
// it bound by the L1 pipe (81 %, 74 % hit rate) at ~10 % of the add-min
// roof.  Here a chunk-column holds 8 columns, so a table row segment is one
// 32-byte sector read by ONE 256-bit load (LDG.E.ENL2.256), and an 8x8 tile
// reuses every loaded value 8 times: per 512 add-mins 16 loads / 16 sectors,
// against 64 loads / 64 half-used sectors for eight 4x4 chunk products.
// Measured (ncu, n = 512, p = 1024): L1 sector traffic per instance drops 4x
// (734 K sectors), but with 255 registers only 8 warps per SM run, and the
// operands -- 48 % L1 hits, the rest from L2 -- leave the kernel waiting on
// long-scoreboard (44 % of stall samples) and barriers (22 %): 6.07 ms
// against 6.33 ms for the 4x4 kernel, slower than it below n ~ 450 (n = 384:
// 2.98 vs 2.61 ms).  Staging each thread's next half chunk in shared memory
// with cp.async (384 threads, 2 stages) measured slower still (8.2 ms), and so
// did L1 prefetches of the next chunk (7.0 ms).  AUTO uses it for n >= 512.
//
// Table: chunk-column m (columns 8m..8m+7) holds rows 0..8m+7, 32 bytes
// each; row-chunk (a, m) starts at word 8*(colbase(m) + a), colbase(m) =
// 4m^2 + 4m.  Before a cell is computed it holds c[a][b] (preloaded).
// Macro tile (I, J), I < J: rows 8I..8I+7, columns 8J..8J+7.  Its k range
//   k in [8I+8, 8J-1]  dense: chunk-columns m = I+1..J-1, split over s lanes
//                      of one warp and min-reduced with xor shuffles;
//   k in (a, 8I+7]     P1: the diagonal tile (I, I) x rows of this tile below;
//   k in [8J, b)       P3: columns of this tile to the left x tile (J, J);
// P1/P3 are an 8x8 triangular solve in registers by the tile's first lane.
// Tile-diagonals D = J - I are processed in order, __syncthreads between.
#include "common.cuh"

#include <climits>

namespace bo {
namespace g8 {

constexpr int kThreads = 256;

template <typename T>
struct __align__(32) V8 { T v[8]; };

template <typename T>
struct Op;
template <>
struct Op<float> {
    static __device__ __forceinline__ float inf() { return __int_as_float(0x7f800000); }
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float min(float a, float b) { return fminf(a, b); }
    // (a + x, a + y): one FADD2 with a broadcast
    static __device__ __forceinline__ float2 add2(float a, float x, float y) {
        return __fadd2_rn(make_float2(a, a), make_float2(x, y));
    }
};
template <>
struct Op<int32_t> {
    static __device__ __forceinline__ int32_t inf() { return INT32_MAX; }
    static __device__ __forceinline__ int32_t add(int32_t a, int32_t b) { return add_wrap(a, b); }
    static __device__ __forceinline__ int32_t min(int32_t a, int32_t b) { return ::min(a, b); }
    static __device__ __forceinline__ int2 add2(int32_t a, int32_t x, int32_t y) {
        return make_int2(add_wrap(a, x), add_wrap(a, y));
    }
};
template <typename T>
__device__ __forceinline__ T min3(T a, T b, T c) { return Op<T>::min(Op<T>::min(a, b), c); }

__host__ __device__ constexpr long long colbase(long long m) { return 4 * m * m + 4 * m; }
__device__ __forceinline__ long long rc(int a, int m) { return 8 * (colbase(m) + a); }   // row-chunk (a, m)
__device__ __forceinline__ long long xo(int a, int b) { return rc(a, b >> 3) + (b & 7); }  // element (a, b)

template <typename T>
__device__ __forceinline__ V8<T> ld8(const T *p) { return *reinterpret_cast<const V8<T> *>(p); }
template <typename T>
__device__ __forceinline__ void st8(T *p, const T (&r)[8]) {
    V8<T> x;
#pragma unroll
    for (int i = 0; i < 8; ++i) x.v[i] = r[i];
    *reinterpret_cast<V8<T> *>(p) = x;
}

// acc[u][v] = min(acc[u][v], min_w A[u].v[w] + B_w[v]) for one 8-wide k chunk;
// B rows (chunk-column J, rows 8m+w) streamed two at a time
__device__ __forceinline__ void chunk(float (&acc)[8][8], const V8<float> (&A)[8], const float *pb) {
#pragma unroll
    for (int w = 0; w < 8; w += 2) {
        const V8<float> B0 = ld8(pb + 8 * w), B1 = ld8(pb + 8 * (w + 1));
#pragma unroll
        for (int u = 0; u < 8; ++u)
#pragma unroll
            for (int v = 0; v < 8; v += 2) {
                const float2 s0 = Op<float>::add2(A[u].v[w], B0.v[v], B0.v[v + 1]);
                const float2 s1 = Op<float>::add2(A[u].v[w + 1], B1.v[v], B1.v[v + 1]);
                acc[u][v] = min3(acc[u][v], s0.x, s1.x);
                acc[u][v + 1] = min3(acc[u][v + 1], s0.y, s1.y);
            }
    }
}
__device__ __forceinline__ void chunk(int32_t (&acc)[8][8], const V8<int32_t> (&A)[8], const int32_t *pb) {
#pragma unroll
    for (int w = 0; w < 8; ++w) {
        const V8<int32_t> B = ld8(pb + 8 * w);
#pragma unroll
        for (int u = 0; u < 8; ++u)
#pragma unroll
            for (int v = 0; v < 8; ++v) acc[u][v] = __viaddmin_s32(A[u].v[w], B.v[v], acc[u][v]);
    }
}

// The 8x8 fix-up of tile (I, J): for u = 7..0,
//   R[v]    = min(S[u][v], min_{w>u} Ad[u][w] + t[w][v])          (P1)
//   t[u][v] = min(R[v], min_{w<v} t[u][w] + Bd[w][v]) + C[u][v]   (P3, in v order)
// Ad / Bd = upper parts of the diagonal tiles (I, I) / (J, J); their entries
// next to the diagonal are polygon edges X[a][a+1] = 0, so those terms are t
// itself (x + 0 == x exactly for the finite non-negative table, G16).
// X[8I+7][8I+8] is an edge too when J = I + 1.
template <typename T>
__device__ __forceinline__ void fixup_store(T *Z, const T (&S)[8][8], int I, int J, bool edge) {
    using O = Op<T>;
    T t[8][8];
    // Bd[w][v] for v > w + 1 (rows 8J..8J+5 of chunk-column J)
    T Bd[6][8];
#pragma unroll
    for (int w = 0; w < 6; ++w) {
        const V8<T> r = ld8(Z + rc(8 * J + w, J));
#pragma unroll
        for (int v = 0; v < 8; ++v) Bd[w][v] = r.v[v];
    }
#pragma unroll
    for (int u = 7; u >= 0; --u) {
        const V8<T> Cu = ld8(Z + rc(8 * I + u, J));            // c[8I+u][8J..8J+7], still in this tile's cells
        T R[8];
        if (u == 7) {
#pragma unroll
            for (int v = 0; v < 8; ++v) R[v] = S[7][v];
        } else {
            const V8<T> Au = ld8(Z + rc(8 * I + u, I));        // Ad[u][w] = X[8I+u][8I+w]
#pragma unroll
            for (int v = 0; v < 8; ++v) R[v] = O::min(S[u][v], t[u + 1][v]);   // w = u+1: Ad = 0
#pragma unroll
            for (int w = u + 2; w < 8; w += 2) {
                if (w + 1 < 8) {
#pragma unroll
                    for (int v = 0; v < 8; v += 2) {
                        const auto x = O::add2(Au.v[w], t[w][v], t[w][v + 1]);
                        const auto y = O::add2(Au.v[w + 1], t[w + 1][v], t[w + 1][v + 1]);
                        R[v] = min3(R[v], x.x, y.x);
                        R[v + 1] = min3(R[v + 1], x.y, y.y);
                    }
                } else {
#pragma unroll
                    for (int v = 0; v < 8; v += 2) {
                        const auto x = O::add2(Au.v[w], t[w][v], t[w][v + 1]);
                        R[v] = O::min(R[v], x.x);
                        R[v + 1] = O::min(R[v + 1], x.y);
                    }
                }
            }
        }
        // P3 in v order: once t[u][w] is final, fold t[u][w] + Bd[w][v] into every v > w + 1
        t[u][0] = (edge && u == 7) ? T(0) : O::add(R[0], Cu.v[0]);
#pragma unroll
        for (int v = 1; v < 8; ++v) {
            const int w = v - 1;                           // Bd[w][w+1] = 0: the term is t[u][w]
#pragma unroll
            for (int x = w + 2; x < 8; ++x) R[x] = O::min(R[x], O::add(t[u][w], Bd[w][x]));
            t[u][v] = O::add(O::min(R[v], t[u][w]), Cu.v[v]);
        }
        st8(Z + rc(8 * I + u, J), t[u]);
    }
}

// Diagonal tile (I, I): the sub-polygon DP on vertices 8I..8I+7 in registers.
template <typename T>
__device__ __forceinline__ void diag_tile(T *Z, int I) {
    using O = Op<T>;
    T X[8][8];
#pragma unroll
    for (int a = 0; a < 8; ++a) {
        const V8<T> r = ld8(Z + rc(8 * I + a, I));
#pragma unroll
        for (int b = 0; b < 8; ++b) X[a][b] = b >= a + 2 ? r.v[b] : T(0);   // c for b >= a+2; edges, below: 0
    }
#pragma unroll
    for (int d = 2; d < 8; ++d)
#pragma unroll
        for (int a = 0; a + d < 8; ++a) {
            const int b = a + d;
            T s = O::add(X[a][a + 1], X[a + 1][b]);
#pragma unroll
            for (int k = a + 2; k < b; ++k) s = O::min(s, O::add(X[a][k], X[k][b]));
            X[a][b] = O::add(s, X[a][b]);
        }
#pragma unroll
    for (int a = 0; a < 8; ++a) st8(Z + rc(8 * I + a, I), X[a]);
}

// lanes per tile on tile-diagonal D (t tiles, D-1 dense chunks, T threads):
// the power of two s <= 32, t*s <= T, that minimises the per-lane chunk count
// (530 instructions each) plus the shuffle reduction (128 per round)
__device__ __forceinline__ int split_log2(int t, int D, int T) {
    int best = 0, cost = (D - 1) * 530;
    for (int l = 1; l <= 5 && (t << l) <= T; ++l) {
        const int c = ((D - 1 + (1 << l) - 1) >> l) * 530 + l * 128;
        if (c < cost) cost = c, best = l;
    }
    return best;
}
}  // namespace g8

template <typename T>
__global__ void __launch_bounds__(g8::kThreads, 1)
tri_global8_kernel(const T *__restrict__ c, T *__restrict__ out, T *ws, int n, long long p, int layout, int NT,
                   int c_vec) {
    pdl_begin();
    using namespace g8;
    using O = Op<T>;
    const long long words = 8 * colbase(NT);
    T *Z = ws + static_cast<long long>(blockIdx.x) * words;
    const int tid = threadIdx.x, nthr = blockDim.x;
    const long long nn = static_cast<long long>(n) * n;
    for (long long i = tid; i < words; i += nthr) Z[i] = T(0);          // padding stays finite
    for (long long h = blockIdx.x; h < p; h += gridDim.x) {
        __syncthreads();
        // 1. weights c[a][b], b >= a+2 -> table (one 32-byte row piece per load)
        if (layout == BO_ROW_WISE && c_vec) {
            const T *ch = c + h * nn;
            for (int idx = tid; idx < (n - 2) * NT; idx += nthr) {
                const int a = idx / NT, m = idx - a * NT;
                if (m >= ((a + 2) >> 3)) *reinterpret_cast<V8<T> *>(Z + rc(a, m)) = ld8(ch + static_cast<long long>(a) * n + 8 * m);
            }
        } else {
            for (int a = 0; a < n - 2; ++a)
                for (int b = a + 2 + tid; b < n; b += nthr) Z[xo(a, b)] = c[tri_c_index(layout, h, n, p, a, b)];
        }
        __syncthreads();
        // 2. D = 0: the diagonal tiles
        for (int I = tid; I < NT; I += nthr) diag_tile(Z, I);
        __syncthreads();
        // 3. tile-diagonals D = 1 .. NT-1
        for (int D = 1; D < NT; ++D) {
            const int t = NT - D;
            const int ls = split_log2(t, D, nthr);
            const int s = 1 << ls;
            for (int base = 0; base < t * s; base += nthr) {           // more tiles than threads: loop
                const int slot = base + tid;
                const int I = slot >> ls, q = slot & (s - 1);
                const bool act = I < t;
                const int J = I + D;
                T acc[8][8];
#pragma unroll
                for (int u = 0; u < 8; ++u)
#pragma unroll
                    for (int v = 0; v < 8; ++v) acc[u][v] = O::inf();
                if (act) {
                    for (int m = I + 1 + q; m < J; m += s) {
                        V8<T> A[8];
#pragma unroll
                        for (int u = 0; u < 8; ++u) A[u] = ld8(Z + rc(8 * I + u, m));
                        chunk(acc, A, Z + rc(8 * m, J));
                    }
                }
                for (int off = 1; off < s; off <<= 1)
#pragma unroll
                    for (int u = 0; u < 8; ++u)
#pragma unroll
                        for (int v = 0; v < 8; ++v) acc[u][v] = O::min(acc[u][v], __shfl_xor_sync(0xffffffffu, acc[u][v], off));
                if (act && q == 0) fixup_store(Z, acc, I, J, D == 1);
            }
            __syncthreads();
        }
        if (tid == 0) out[h] = Z[xo(0, n - 1)];
    }
}

size_t tiled_global8_workspace(int64_t n, int64_t p) {
    const long long NT = (n + 7) / 8;
    const long long grid = std::min<long long>(p, num_sms());
    return static_cast<size_t>(grid) * 8 * g8::colbase(NT) * 4;
}

int launch_tri_global8(const void *c, void *out, void *ws, int64_t n, int64_t p, int dtype, int layout,
                       cudaStream_t st) {
    const int NT = static_cast<int>((n + 7) / 8);
    const long long grid = std::min<long long>(p, num_sms());
    if ((reinterpret_cast<uintptr_t>(ws) & 31u) != 0) return fail(BO_EINVAL, "TILED_GLOBAL8: workspace must be 32-byte aligned");
    const int c_vec = (n % 8 == 0) && (reinterpret_cast<uintptr_t>(c) & 31u) == 0;
    if (dtype == BO_F32)
        launch(tri_global8_kernel<float>, static_cast<unsigned>(grid), g8::kThreads, 0, st, static_cast<const float *>(c),
               static_cast<float *>(out), static_cast<float *>(ws), static_cast<int>(n), p, layout, NT, c_vec);
    else
        launch(tri_global8_kernel<int32_t>, static_cast<unsigned>(grid), g8::kThreads, 0, st,
               static_cast<const int32_t *>(c), static_cast<int32_t *>(out), static_cast<int32_t *>(ws),
               static_cast<int>(n), p, layout, NT, c_vec);
    return after_launch("tri_global8_kernel");
}

}  // namespace bo
