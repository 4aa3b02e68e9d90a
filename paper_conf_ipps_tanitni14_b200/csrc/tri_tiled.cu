// tri_tiled.cu -- blocked min-plus evaluation of Algorithm OPT:
// LPI lanes per instance (16 or 32), table in shared memory, 4x4 register
// tiles.  Bit-identical to the sequential algorithm (see tri.cu header).
//
// Vertex coordinates.  With X[r][j] := M[r+1][j] (the paper's M over the
// sub-polygon v_r..v_j), Algorithm OPT's update
//   M[i,j] = min_{k=i}^{j-1} (M[i,k] + M[k+1,j]) + c[i-1,j]
// reads, for 0 <= a < b <= n-1,
//   X[a][a+1] = 0,   X[a][b] = min_{a<k<b} (X[a][k] + X[k][b]) + c[a][b],
// the same sums in the same association, and out = X[0][n-1] = M[1,n-1].
// c[a][b] and X[a][b] share coordinates, so c is preloaded into the table.
//
// Shared-memory table Z (NP = 4*ceil(n/4) rows, row stride 68 elements):
//   Z[a][b] = X[a][b] for b > a (initially c[a][b]),  Z[b][a] = X[a][b].
// For a tile (I,J), I < J (rows 4I..4I+3, cols 4J..4J+3) the k range splits
//   k in [4I+4, 4J-1]  -> min-plus "dot product" of row-blocks I and J of Z
//                         over aligned 4-wide column chunks m = I+1..J-1:
//                         S[u][v] = min_m min_w Z[4I+u][4m+w] + Z[4J+v][4m+w]
//   k in (a, 4I+3]     -> P1: diagonal tile (I,I) x rows of this tile below
//   k in [4J, b)       -> P3: columns of this tile to the left x tile (J,J)
// One chunk = 8 LDS.128 + 64 add-mins; consecutive k sit in adjacent
// registers, so fp32 runs as FADD2 + FMNMX3 (one instruction per add-min)
// and int32 as VIADDMNMX.  P1/P3 are a 4x4 triangular solve in registers.
// Tiles of one tile-diagonal D = J-I are independent; long dense ranges are
// split over s lanes and min-reduced with xor shuffles.  Row stride 68 puts
// chunk m of row r in bank group (r + m) mod 8 and keeps a tile's four rows
// at immediate offsets.
#include "common.cuh"

#include <climits>

namespace bo {

namespace tt {
template <typename T>
struct Ops;
template <>
struct Ops<float> {
    static __device__ __forceinline__ float inf() { return __int_as_float(0x7f800000); }
    static __device__ __forceinline__ float add(float a, float b) { return __fadd_rn(a, b); }
    static __device__ __forceinline__ float min(float a, float b) { return fminf(a, b); }
    static __device__ __forceinline__ float addmin(float a, float b, float s) { return fminf(__fadd_rn(a, b), s); }
    // min(s, a.x + b.x, a.y + b.y): FADD2 + FMNMX3
    static __device__ __forceinline__ float addmin2(float2 a, float2 b, float s) {
        const float2 r = __fadd2_rn(a, b);
        return fminf(fminf(s, r.x), r.y);
    }
};
template <>
struct Ops<int32_t> {
    static __device__ __forceinline__ int32_t inf() { return INT32_MAX; }
    static __device__ __forceinline__ int32_t add(int32_t a, int32_t b) { return add_wrap(a, b); }
    static __device__ __forceinline__ int32_t min(int32_t a, int32_t b) { return ::min(a, b); }
    static __device__ __forceinline__ int32_t addmin(int32_t a, int32_t b, int32_t s) {
        return __viaddmin_s32(a, b, s);
    }
    static __device__ __forceinline__ int32_t addmin2(int2 a, int2 b, int32_t s) {
        return __viaddmin_s32(a.y, b.y, __viaddmin_s32(a.x, b.x, s));
    }
};
template <typename T> struct V2;
template <> struct V2<float> { using type = float2; };
template <> struct V2<int32_t> { using type = int2; };
template <typename T> struct V4;
template <> struct V4<float> { using type = float4; };
template <> struct V4<int32_t> { using type = int4; };

constexpr int kRS = 68;   // row stride (elements)

template <typename T>
__device__ __forceinline__ typename V4<T>::type ld4(const T *p) {
    return *reinterpret_cast<const typename V4<T>::type *>(p);
}
template <typename T>
__device__ __forceinline__ void st4(T *p, T x, T y, T z, T w) {
    typename V4<T>::type v;
    v.x = x; v.y = y; v.z = z; v.w = w;
    *reinterpret_cast<typename V4<T>::type *>(p) = v;
}
__device__ __forceinline__ void cp_async16(void *dst, const void *src, bool pred) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t"
        "@p cp.async.cg.shared.global [%0], [%1], 16;\n\t}" ::"r"(smem_u32(dst)),
        "l"(src), "r"(static_cast<int>(pred))
        : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// 16 partial tiles: consecutive k pairs (w, w+1) come from one 128-bit load
template <typename T>
__device__ __forceinline__ void minplus_chunk(T (&acc)[4][4], const typename V4<T>::type (&A)[4],
                                              const typename V4<T>::type (&B)[4]) {
    using T2 = typename V2<T>::type;
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const T x = Ops<T>::addmin2(T2{A[u].x, A[u].y}, T2{B[v].x, B[v].y}, acc[u][v]);
            acc[u][v] = Ops<T>::addmin2(T2{A[u].z, A[u].w}, T2{B[v].z, B[v].w}, x);
        }
}
}  // namespace tt

// Lanes per tile on tile-diagonal D (t = NT-D tiles): 2^ls, the largest power
// of two with t * 2^ls <= lanes that does not exceed the D-1 dense chunks.
__device__ __forceinline__ int split_log2(int t, int D, int lpi) {
    int ls = 0;
    while ((2 << ls) * t <= lpi && (1 << ls) < D - 1) ++ls;
    return ls;
}

template <typename T, int LPI>
__global__ void __launch_bounds__(128, 1)
tri_tiled_kernel(const T *__restrict__ c, T *__restrict__ out, int n, long long p, int layout, int NT, int c_vec) {
    using Op = tt::Ops<T>;
    using T4 = typename tt::V4<T>::type;
    using tt::kRS;
    constexpr int IPW = 32 / LPI;                       // instances per warp
    extern __shared__ uint8_t smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int slot = lane / LPI, li = lane % LPI;       // instance slot in warp, lane in instance
    const int NP = 4 * NT;
    const int warps_per_cta = blockDim.x >> 5;
    T *Z = reinterpret_cast<T *>(smem_raw) + static_cast<size_t>(warp * IPW + slot) * NP * kRS;

    // zero the table once: padding rows / columns then stay finite forever
    for (int i = li; i < NP * kRS; i += LPI) Z[i] = T(0);
    __syncwarp();

    const long long inst_stride = static_cast<long long>(gridDim.x) * warps_per_cta * IPW;
    const long long nn = static_cast<long long>(n) * n;
    const int last_chunk = (n - 1) >> 2;

    for (long long h = (static_cast<long long>(blockIdx.x) * warps_per_cta + warp) * IPW + slot;
         h - slot < p; h += inst_stride) {
        const bool live = h < p;
        // ------------------------------------------------ 1. c -> upper table
        // Only the weights Algorithm OPT reads (b >= a+2) are fetched.
        if (layout == BO_ROW_WISE && c_vec) {
            const T *ch = c + (live ? h : 0) * nn;
            // warm L2 with the next instance this lane group will process: only the
            // row segments Algorithm OPT reads (b >= a+2), one bulk prefetch per row
            if (h + inst_stride < p) {
                const T *cn = c + (h + inst_stride) * nn;
                for (int a = li; a < n - 2; a += LPI) {
                    const int m0 = (a + 2) >> 2;
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cn + static_cast<long long>(a) * n + 4 * m0),
                                 "r"(static_cast<unsigned>((n - 4 * m0) * sizeof(T)))
                                 : "memory");
                }
            }
            // lane li copies chunk m0(a)+li of row a; LPI=32 handles two rows per step
            for (int a0 = 0; a0 < n - 2; a0 += LPI / 16) {
                const int a = a0 + (li >> 4);
                const int m = ((a + 2) >> 2) + (li & 15);
                tt::cp_async16(Z + a * kRS + 4 * m, ch + static_cast<long long>(a) * n + 4 * m,
                           live && a < n - 2 && m <= last_chunk);
            }
            tt::cp_async_wait_all();
        } else if (live) {
            for (int a = 0; a < n - 2; ++a)
                for (int b = a + 2 + li; b < n; b += LPI)
                    Z[a * kRS + b] = __ldg(c + (layout == BO_ROW_WISE ? h * nn + static_cast<long long>(a) * n + b
                                                                      : (static_cast<long long>(a) * n + b) * p + h));
        }
        __syncwarp();

        // ------------------------------------------------ 2. D = 0 (diagonal tiles)
        if (li < NT) {
            const int I = li;
            T *r0 = Z + (4 * I) * kRS + 4 * I;
            const T4 c0 = tt::ld4(r0), c1 = tt::ld4(r0 + kRS);
            const T z = T(0);
            // X[a][a+1] = 0; X[0][2], X[1][3] have the single k with two zero terms
            const T t02 = Op::add(Op::add(z, z), c0.z);
            const T t13 = Op::add(Op::add(z, z), c1.w);
            const T t03 = Op::add(Op::min(Op::add(z, t13), Op::add(t02, z)), c0.w);
            tt::st4(r0, z, z, t02, t03);
            tt::st4(r0 + kRS, z, z, z, t13);
            tt::st4(r0 + 2 * kRS, t02, z, z, z);
            tt::st4(r0 + 3 * kRS, t03, t13, z, z);
        }
        __syncwarp();

        // ------------------------------------------------ 3. D = 1 .. NT-1
        for (int D = 1; D < NT; ++D) {
            const int ls = split_log2(NT - D, D, LPI);
            const int s = 1 << ls;
            const int I = li >> ls, q = li & (s - 1);
            const bool act = I < NT - D;
            const int J = I + D;
            T acc[4][4];
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) acc[u][v] = Op::inf();
            if (act) {
                int m = I + 1 + q;
                const T *pa = Z + (4 * I) * kRS + 4 * m;
                const T *pb = Z + (4 * J) * kRS + 4 * m;
                if (m < J) {
                    // software-pipelined ping-pong: load chunk m+s while computing chunk m
                    T4 A0[4], B0[4], A1[4], B1[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) A0[u] = tt::ld4(pa + u * kRS), B0[u] = tt::ld4(pb + u * kRS);
                    while (true) {
                        m += s;
                        pa += 4 * s;
                        pb += 4 * s;
                        bool more = m < J;
                        if (more) {
#pragma unroll
                            for (int u = 0; u < 4; ++u) A1[u] = tt::ld4(pa + u * kRS), B1[u] = tt::ld4(pb + u * kRS);
                        }
                        tt::minplus_chunk<T>(acc, A0, B0);
                        if (!more) break;
                        m += s;
                        pa += 4 * s;
                        pb += 4 * s;
                        more = m < J;
                        if (more) {
#pragma unroll
                            for (int u = 0; u < 4; ++u) A0[u] = tt::ld4(pa + u * kRS), B0[u] = tt::ld4(pb + u * kRS);
                        }
                        tt::minplus_chunk<T>(acc, A1, B1);
                        if (!more) break;
                    }
                }
            }
            for (int off = 1; off < s; off <<= 1)
#pragma unroll
                for (int u = 0; u < 4; ++u)
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        acc[u][v] = Op::min(acc[u][v], __shfl_xor_sync(0xffffffffu, acc[u][v], off));
            if (act && q == 0) {
                // A[u][w] = X[4I+u][4I+w] (w > u), Bd[w][v] = X[4J+w][4J+v] (v > w),
                // C[u][v] = c[4I+u][4J+v] (still in the tile's own upper cells)
                T *ta = Z + (4 * I) * kRS + 4 * I;
                T *tb = Z + (4 * J) * kRS + 4 * J;
                T *tc = Z + (4 * I) * kRS + 4 * J;
                T A[4][4], Bd[4][4], C[4][4];
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    const T4 x = tt::ld4(ta + r * kRS), y = tt::ld4(tb + r * kRS), w = tt::ld4(tc + r * kRS);
                    A[r][0] = x.x; A[r][1] = x.y; A[r][2] = x.z; A[r][3] = x.w;
                    Bd[r][0] = y.x; Bd[r][1] = y.y; Bd[r][2] = y.z; Bd[r][3] = y.w;
                    C[r][0] = w.x; C[r][1] = w.y; C[r][2] = w.z; C[r][3] = w.w;
                }
                T t[4][4];
#pragma unroll
                for (int u = 3; u >= 0; --u)
#pragma unroll
                    for (int v = 0; v < 4; ++v) {
                        T sv = acc[u][v];
#pragma unroll
                        for (int w = u + 1; w < 4; ++w) sv = Op::addmin(A[u][w], t[w][v], sv);   // P1
#pragma unroll
                        for (int w = 0; w < v; ++w) sv = Op::addmin(t[u][w], Bd[w][v], sv);       // P3
                        t[u][v] = Op::add(sv, C[u][v]);
                        // X[4I+3][4I+4] is an edge of the polygon (M[i][i] = 0)
                        if (u == 3 && v == 0 && D == 1) t[u][v] = T(0);
                    }
#pragma unroll
                for (int u = 0; u < 4; ++u) tt::st4(tc + u * kRS, t[u][0], t[u][1], t[u][2], t[u][3]);
                T *tl = Z + (4 * J) * kRS + 4 * I;      // transpose into the lower part
#pragma unroll
                for (int v = 0; v < 4; ++v) tt::st4(tl + v * kRS, t[0][v], t[1][v], t[2][v], t[3][v]);
            }
            __syncwarp();
        }
        if (live && li == 0) out[h] = Z[n - 1];          // X[0][n-1] = Algorithm OPT's M[1,n-1]
        __syncwarp();
    }
}

int tiled_supported(int64_t n) { return n >= 5 && n <= 64; }

template <typename T, int LPI>
static int launch_tiled_t(const void *c, void *out, int64_t n, int64_t p, int layout, cudaStream_t st) {
    const int NT = static_cast<int>((n + 3) / 4);
    const size_t per_inst = static_cast<size_t>(4 * NT) * tt::kRS * sizeof(T);
    constexpr int IPW = 32 / LPI;
    // warps per CTA: the W in 1..4 that keeps the most warps resident per SM
    // (shared memory is the limit: 227 KB, 1 KB reserved per CTA)
    int W = 1, best = 0;
    for (int w = 1; w <= 4; ++w) {
        const size_t per_cta = w * IPW * per_inst + 1024;
        const int resident = static_cast<int>((227 * 1024) / per_cta) * w;
        if (resident > best) best = resident, W = w;
    }
    const size_t smem = W * IPW * per_inst;
    static bool attr = [] {
        return cudaFuncSetAttribute(tri_tiled_kernel<T, LPI>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    227 * 1024) == cudaSuccess;
    }();
    if (!attr) return fail(BO_ECUDA, "tiled: cannot set dynamic smem");
    int per_sm = 1;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, tri_tiled_kernel<T, LPI>, W * 32, smem);
    per_sm = std::max(per_sm, 1);
    const long long per_cta = static_cast<long long>(W) * IPW;
    const long long blocks = std::min<long long>((p + per_cta - 1) / per_cta,
                                                 static_cast<long long>(per_sm) * num_sms());
    const int c_vec = (n % 4 == 0) && aligned16(c);
    tri_tiled_kernel<T, LPI><<<static_cast<unsigned>(blocks), W * 32, smem, st>>>(
        static_cast<const T *>(c), static_cast<T *>(out), static_cast<int>(n), p, layout, NT, c_vec);
    return after_launch("tri_tiled_kernel");
}

// lpi: lanes per instance (BO_TRI_TILED = 32, BO_TRI_TILED_HALF = 16)
int launch_tri_tiled(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout, int lpi,
                     cudaStream_t st) {
    if (dtype == BO_F32)
        return lpi == 16 ? launch_tiled_t<float, 16>(c, out, n, p, layout, st)
                         : launch_tiled_t<float, 32>(c, out, n, p, layout, st);
    return lpi == 16 ? launch_tiled_t<int32_t, 16>(c, out, n, p, layout, st)
                     : launch_tiled_t<int32_t, 32>(c, out, n, p, layout, st);
}

}  // namespace bo
