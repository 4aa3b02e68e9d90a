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
// Shared-memory table: the UPPER triangle only, stored by 4-wide column
// chunks ("chunk-columns"): chunk-column m holds rows 0..4m+3 (+1 pad row) of
// columns 4m..4m+3, so element X[a][b] lives at chunk colbase(b/4) + a, word
// b%4, with colbase(m) = 2m^2 + 3m (heights 4m+5 are odd, which spreads the
// quarter-warp's chunks over all 8 bank groups).  8.75 KB per instance at
// n = 64 instead of a 16 KB square, so twice as many instances per SM.
// Before a cell is computed it holds c[a][b] (preloaded with cp.async).
// For a tile (I,J), I < J (rows 4I..4I+3, cols 4J..4J+3) the k range splits
//   k in [4I+4, 4J-1]  -> dense min-plus product over chunk-columns m = I+1..J-1:
//                         A_u = X[4I+u][4m..4m+3]   (chunk-column m, rows 4I+u)
//                         B_w = X[4m+w][4J..4J+3]   (chunk-column J, rows 4m+w)
//                         S[u][v] = min_w A_u[w] + B_w[v]
//   k in (a, 4I+3]     -> P1: diagonal tile (I,I) x rows of this tile below
//   k in [4J, b)       -> P3: columns of this tile to the left x tile (J,J)
// One chunk = 8 LDS.128 (each row read at an immediate offset) + 64
// add-mins; fp32 pairs two v's in one FADD2 with the A value broadcast
// (FADD2 Rd, Ra.F32, Rb.F32x2) and folds two k's per FMNMX3 -- one
// instruction per add-min; int32 is one VIADDMNMX per add-min.  P1/P3 are
// a 4x4 triangular solve in registers ("fix-up").  Tiles of one
// tile-diagonal D = J-I are independent; long dense ranges are split over s
// lanes and min-reduced with xor shuffles.
#include "common.cuh"

#include <climits>

namespace bo {

#ifdef BO_TRI_CLOCK
// development instrumentation: cycles per phase (slot 0 = preload, 1 = D=0,
// 1+D = tile-diagonal D), summed over the instances of lane 0 of every warp
__device__ unsigned long long g_tri_clock[160];   // 80 + 4D + k: sub-phases of step D
#define BO_CLK_MARK(slot)                                                             \
    do {                                                                              \
        const long long t_ = clock64();                                               \
        if (lane == 0) atomicAdd(&g_tri_clock[(slot)], static_cast<unsigned long long>(t_ - clk_)); \
        clk_ = clock64();                                                             \
    } while (0)
#else
#define BO_CLK_MARK(slot) do {} while (0)
#endif

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

// chunk-column m starts at chunk colbase(m); element (a, b) at word xoff(a, b)
__host__ __device__ __forceinline__ constexpr int colbase(int m) { return 2 * m * m + 3 * m; }
__device__ __forceinline__ int xc(int a, int m) { return 4 * (colbase(m) + a); }   // chunk (row a, col-chunk m)
__device__ __forceinline__ int xoff(int a, int b) { return xc(a, b >> 2) + (b & 3); }

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
__device__ __forceinline__ void cp_async4(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }
// S[u][v] = min(S[u][v], min_w A[u].w + B[w].v) for one 4-wide k chunk
__device__ __forceinline__ float comp(const float4 &v, int i) { return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w; }
__device__ __forceinline__ int comp(const int4 &v, int i) { return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w; }

__device__ __forceinline__ void minplus_chunk(float (&acc)[4][4], const float4 (&A)[4], const float4 (&B)[4]) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int w = 0; w < 4; w += 2) {
            const float a0 = comp(A[u], w), a1 = comp(A[u], w + 1);
#pragma unroll
            for (int v = 0; v < 4; v += 2) {
                const float2 s0 = __fadd2_rn(make_float2(a0, a0), make_float2(comp(B[w], v), comp(B[w], v + 1)));
                const float2 s1 = __fadd2_rn(make_float2(a1, a1), make_float2(comp(B[w + 1], v), comp(B[w + 1], v + 1)));
                acc[u][v] = fminf(fminf(acc[u][v], s0.x), s1.x);
                acc[u][v + 1] = fminf(fminf(acc[u][v + 1], s0.y), s1.y);
            }
        }
}
// acc = the first chunk's min_w A[u].w + B[w].v (same sums, min order is free)
__device__ __forceinline__ void minplus_first(float (&acc)[4][4], const float4 (&A)[4], const float4 (&B)[4]) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; v += 2) {
            float2 s[4];
#pragma unroll
            for (int w = 0; w < 4; ++w) {
                const float a = comp(A[u], w);
                s[w] = __fadd2_rn(make_float2(a, a), make_float2(comp(B[w], v), comp(B[w], v + 1)));
            }
            acc[u][v] = fminf(fminf(fminf(s[0].x, s[1].x), s[2].x), s[3].x);
            acc[u][v + 1] = fminf(fminf(fminf(s[0].y, s[1].y), s[2].y), s[3].y);
        }
}
__device__ __forceinline__ void minplus_first(int32_t (&acc)[4][4], const int4 (&A)[4], const int4 (&B)[4]) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            int32_t r = add_wrap(comp(A[u], 0), comp(B[0], v));
#pragma unroll
            for (int w = 1; w < 4; ++w) r = __viaddmin_s32(comp(A[u], w), comp(B[w], v), r);
            acc[u][v] = r;
        }
}
__device__ __forceinline__ void minplus_chunk(int32_t (&acc)[4][4], const int4 (&A)[4], const int4 (&B)[4]) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int w = 0; w < 4; ++w)
#pragma unroll
            for (int v = 0; v < 4; ++v) acc[u][v] = __viaddmin_s32(comp(A[u], w), comp(B[w], v), acc[u][v]);
}
// The 4x4 fix-up of one tile: with S = the dense part (k outside the tile's
// own diagonal tiles), for u = 3..0, v = 0..3
//   t[u][v] = min(S[u][v], min_{w>u} A[u][w] + t[w][v]   (P1, diagonal tile I)
//                         , min_{w<v} t[u][w] + Bd[w][v]) (P3, diagonal tile J)
//             + C[u][v]
// -- the same sums as Algorithm OPT's inner loop, min taken in another order
// (exact).  Generic form: one add-min per term.
template <typename T>
__device__ __forceinline__ void fixup(T (&t)[4][4], const T (&S)[4][4], const T (&A)[4][4], const T (&Bd)[4][4],
                                      const T (&C)[4][4], bool edge) {
#pragma unroll
    for (int u = 3; u >= 0; --u)
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            T sv = S[u][v];
#pragma unroll
            for (int w = u + 1; w < 4; ++w) sv = Ops<T>::addmin(A[u][w], t[w][v], sv);   // P1
#pragma unroll
            for (int w = 0; w < v; ++w) sv = Ops<T>::addmin(t[u][w], Bd[w][v], sv);       // P3
            t[u][v] = Ops<T>::add(sv, C[u][v]);
            if (u == 3 && v == 0 && edge) t[u][v] = T(0);
        }
}
__device__ __forceinline__ float2 add2b(float a, float x, float y) {
    return __fadd2_rn(make_float2(a, a), make_float2(x, y));
}
__device__ __forceinline__ float min3(float a, float b, float c) { return fminf(fminf(a, b), c); }
// fp32, row-ordered: P1 terms of a row pair two v's in one FADD2 (A[u][w]
// broadcast), mins fold two terms per FMNMX3, and the polygon edges X[a][a+1]
// of the diagonal tiles are 0 (M[i][i] = 0): A[u][u+1] =
// Bd[w][w+1] = 0, so those terms are t itself (x + 0 == x exactly for the
// finite, non-negative values of the table, G16) -- 14 instructions less per
// tile than the plain pairing, and Bd rows 2..3 are never read.  (A
// latency-ordered variant -- cells by anti-diagonal, newest terms last,
// scalar adds -- measured 5% slower: the kernel is bound by issue slots more
// than by this chain.)
template <>
__device__ __forceinline__ void fixup<float>(float (&t)[4][4], const float (&S)[4][4], const float (&A)[4][4],
                                             const float (&Bd)[4][4], const float (&C)[4][4], bool edge) {
    float R[4];
    // u = 3: no P1 term
#pragma unroll
    for (int v = 0; v < 4; ++v) R[v] = S[3][v];
    auto p3 = [&](int u) {
        t[u][0] = edge && u == 3 ? 0.0f : __fadd_rn(R[0], C[u][0]);
        const float2 a23 = add2b(t[u][0], Bd[0][2], Bd[0][3]);
        t[u][1] = __fadd_rn(fminf(R[1], t[u][0]), C[u][1]);
        const float b3 = __fadd_rn(t[u][1], Bd[1][3]);
        t[u][2] = __fadd_rn(min3(R[2], a23.x, t[u][1]), C[u][2]);
        t[u][3] = __fadd_rn(min3(fminf(R[3], a23.y), b3, t[u][2]), C[u][3]);
    };
    p3(3);
    // u = 2: w = 3 (A = 0)
#pragma unroll
    for (int v = 0; v < 4; ++v) R[v] = fminf(S[2][v], t[3][v]);
    p3(2);
    // u = 1: w = 2 (A = 0), w = 3
    {
        const float2 y01 = add2b(A[1][3], t[3][0], t[3][1]), y23 = add2b(A[1][3], t[3][2], t[3][3]);
        R[0] = min3(S[1][0], t[2][0], y01.x); R[1] = min3(S[1][1], t[2][1], y01.y);
        R[2] = min3(S[1][2], t[2][2], y23.x); R[3] = min3(S[1][3], t[2][3], y23.y);
    }
    p3(1);
    // u = 0: w = 1 (A = 0), w = 2, w = 3
    {
        const float2 y01 = add2b(A[0][2], t[2][0], t[2][1]), y23 = add2b(A[0][2], t[2][2], t[2][3]);
        const float2 z01 = add2b(A[0][3], t[3][0], t[3][1]), z23 = add2b(A[0][3], t[3][2], t[3][3]);
        R[0] = fminf(min3(S[0][0], t[1][0], y01.x), z01.x);
        R[1] = fminf(min3(S[0][1], t[1][1], y01.y), z01.y);
        R[2] = fminf(min3(S[0][2], t[1][2], y23.x), z23.x);
        R[3] = fminf(min3(S[0][3], t[1][3], y23.y), z23.y);
    }
    p3(0);
}

// Dense part of tile (I, J) over chunk-columns m, m + s, ... < J (m < J):
// software-pipelined ping-pong (load chunk m+s while computing chunk m); acc
// arrives filled with +inf.
template <typename T>
__device__ __forceinline__ void dense_tile(T (&acc)[4][4], const T *Z, int I, int J, int m, int s) {
    using T4 = typename V4<T>::type;
    const T *pa = Z + xc(4 * I, m);                 // A rows 4I+u: pa + 4u
    const T *pb = Z + xc(4 * m, J);                 // B rows 4m+w: pb + 4w
    const int db = 16 * s;                          // B: next chunk = 4s rows further down
    T4 A0[4], B0[4], A1[4], B1[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) A0[u] = ld4(pa + 4 * u), B0[u] = ld4(pb + 4 * u);
    pa += 4 * (4 * m * s + 2 * s * s + 3 * s);       // colbase(m+s) - colbase(m) chunks
    pb += db;
    m += s;
    bool more = m < J;
    if (more) {
#pragma unroll
        for (int u = 0; u < 4; ++u) A1[u] = ld4(pa + 4 * u), B1[u] = ld4(pb + 4 * u);
    }
    minplus_chunk(acc, A0, B0);
    while (more) {
        pa += 4 * (4 * m * s + 2 * s * s + 3 * s);
        pb += db;
        m += s;
        more = m < J;
        if (more) {
#pragma unroll
            for (int u = 0; u < 4; ++u) A0[u] = ld4(pa + 4 * u), B0[u] = ld4(pb + 4 * u);
        }
        minplus_chunk(acc, A1, B1);
        if (!more) break;
        pa += 4 * (4 * m * s + 2 * s * s + 3 * s);
        pb += db;
        m += s;
        more = m < J;
        if (more) {
#pragma unroll
            for (int u = 0; u < 4; ++u) A1[u] = ld4(pa + 4 * u), B1[u] = ld4(pb + 4 * u);
        }
        minplus_chunk(acc, A0, B0);
    }
}
// Two tiles (I0, I0+D), (I1, I1+D) of one tile-diagonal, all D-1 chunks each
// (s = 1), interleaved; D == 1 has no dense chunk (acc = +inf).
template <typename T>
__device__ __forceinline__ void dense_tile2(T (&acc0)[4][4], T (&acc1)[4][4], const T *Z, int I0, int I1, int D) {
    using T4 = typename V4<T>::type;
    if (D < 2) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v) acc0[u][v] = acc1[u][v] = Ops<T>::inf();
        return;
    }
    int m0 = I0 + 1, m1 = I1 + 1;
    const T *pa0 = Z + xc(4 * I0, m0), *pb0 = Z + xc(4 * m0, I0 + D);
    const T *pa1 = Z + xc(4 * I1, m1), *pb1 = Z + xc(4 * m1, I1 + D);
    T4 A0[4], B0[4], A1[4], B1[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) A0[u] = ld4(pa0 + 4 * u), B0[u] = ld4(pb0 + 4 * u);
#pragma unroll
    for (int u = 0; u < 4; ++u) A1[u] = ld4(pa1 + 4 * u), B1[u] = ld4(pb1 + 4 * u);
    minplus_first(acc0, A0, B0);
    minplus_first(acc1, A1, B1);
    for (int k = 2; k < D; ++k) {
        pa0 += 4 * (4 * m0 + 5), pa1 += 4 * (4 * m1 + 5);       // colbase(m+1) - colbase(m) = 4m + 5 chunks
        pb0 += 16, pb1 += 16;
        ++m0, ++m1;
#pragma unroll
        for (int u = 0; u < 4; ++u) A0[u] = ld4(pa0 + 4 * u), B0[u] = ld4(pb0 + 4 * u);
#pragma unroll
        for (int u = 0; u < 4; ++u) A1[u] = ld4(pa1 + 4 * u), B1[u] = ld4(pb1 + 4 * u);
        minplus_chunk(acc0, A0, B0);
        minplus_chunk(acc1, A1, B1);
    }
}
// The upper part of a diagonal tile (I, I) after step D = 0:
// X[4I][4I+1..3] = (0, t02, t03), X[4I+1][4I+2..3] = (0, t13), X[4I+2][4I+3] = 0.
// The lane that fixes up row block I (lane I) computed it itself and keeps it
// in registers (d[0..2] = t02, t03, t13) instead of reloading it every step.
template <typename T>
__device__ __forceinline__ void diag_upper(T (&A)[4][4], const T (&d)[3]) {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) A[u][v] = T(0);
    A[0][2] = d[0]; A[0][3] = d[1]; A[1][3] = d[2];
}
template <typename T>
__device__ __forceinline__ void load_fix_operands(const T *Z, int I, int J, const T (&d)[3], T (&A)[4][4],
                                                  T (&Bd)[4][4], T (&C)[4][4]) {
    using T4 = typename V4<T>::type;
    // A[u][w] = X[4I+u][4I+w] (w > u; registers), Bd[w][v] = X[4J+w][4J+v] (v > w),
    // C[u][v] = c[4I+u][4J+v] (still in the tile's own upper cells)
    diag_upper(A, d);
    const T *tb = Z + xc(4 * J, J), *tc = Z + xc(4 * I, J);
#pragma unroll
    for (int r = 0; r < 4; ++r) {
        const T4 y = ld4(tb + 4 * r), w = ld4(tc + 4 * r);
        Bd[r][0] = y.x; Bd[r][1] = y.y; Bd[r][2] = y.z; Bd[r][3] = y.w;
        C[r][0] = w.x; C[r][1] = w.y; C[r][2] = w.z; C[r][3] = w.w;
    }
}
// fix-up of tile (I, J = I + D) and store; X[4I+3][4I+4] is an edge of the
// polygon when D == 1 (M[i][i] = 0)
template <typename T>
__device__ __forceinline__ void finish_tile(T *Z, const T (&acc)[4][4], int I, int J, int D, const T (&d)[3]) {
    T A[4][4], Bd[4][4], C[4][4], t[4][4];
    load_fix_operands(Z, I, J, d, A, Bd, C);
    fixup(t, acc, A, Bd, C, D == 1);
    T *tc = Z + xc(4 * I, J);
#pragma unroll
    for (int u = 0; u < 4; ++u) st4(tc + 4 * u, t[u][0], t[u][1], t[u][2], t[u][3]);
}
template <typename T>
__device__ __forceinline__ void finish_tile2(T *Z, const T (&acc0)[4][4], const T (&acc1)[4][4], int I0, int I1, int D,
                                             bool st1, const T (&d0)[3], const T (&d1)[3]) {
    T A0[4][4], Bd0[4][4], C0[4][4], t0[4][4], A1[4][4], Bd1[4][4], C1[4][4], t1[4][4];
    load_fix_operands(Z, I0, I0 + D, d0, A0, Bd0, C0);
    load_fix_operands(Z, I1, I1 + D, st1 ? d1 : d0, A1, Bd1, C1);
    fixup(t0, acc0, A0, Bd0, C0, D == 1);
    fixup(t1, acc1, A1, Bd1, C1, D == 1);
    T *tc0 = Z + xc(4 * I0, I0 + D), *tc1 = Z + xc(4 * I1, I1 + D);
#pragma unroll
    for (int u = 0; u < 4; ++u) st4(tc0 + 4 * u, t0[u][0], t0[u][1], t0[u][2], t0[u][3]);
    if (st1) {
#pragma unroll
        for (int u = 0; u < 4; ++u) st4(tc1 + 4 * u, t1[u][0], t1[u][1], t1[u][2], t1[u][3]);
    }
}
}  // namespace tt

// Lanes per tile on tile-diagonal D (t = NT-D tiles): 2^ls, the largest power
// of two with t * 2^ls <= lanes that does not exceed the D-1 dense chunks.
__host__ __device__ inline int split_log2(int t, int D, int lpi) {
    int ls = 0;
    while ((2 << ls) * t <= lpi && (1 << ls) < D - 1) ++ls;
    return ls;
}
// the whole schedule in one kernel parameter: 4 bits of log2(split) per D
static uint64_t split_schedule(int NT, int lpi) {
    // (measured: requiring >= 3 or 4 chunks per split lane -- fewer shuffle
    // rounds, longer dense runs -- is 2-6% slower at n = 64)
    uint64_t m = 0;
    for (int D = 1; D < NT; ++D) m |= static_cast<uint64_t>(split_log2(NT - D, D, lpi)) << (4 * D);
    return m;
}

// Shared words between consecutive instance tables.  Two instances per warp
// (LPI = 16) sit on alternate lanes (slot = lane & 1), so an 8-lane LDS.128
// phase holds 4 tiles of each; their tables are offset by 16 words (mod 32)
// so the two halves fall in opposite bank-group halves (tools/smem_model.py,
// --interleave: 1124 -> 968 wavefronts per instance at n = 64).
// Four instances per warp (LPI = 8) sit on lanes = slot mod 4 with tables
// 8 words (mod 32) apart, the same idea one level down.
__host__ __device__ constexpr int table_stride(int NT, int ipw) {
    return ipw > 1 ? 4 * (2 * NT * NT + 3 * NT) + ((32 / ipw - 4 * (2 * NT * NT + 3 * NT)) % 32 + 32) % 32
                   : 4 * (2 * NT * NT + 3 * NT);
}

// Step 1 of an instance: c -> upper table.  Only the weights Algorithm OPT
// reads (b >= a+2) are fetched; waits for its own copies.
template <typename T, int LPI, bool WAIT = true>
__device__ __forceinline__ void preload_table(T *Z, const T *__restrict__ c, long long h, bool live, int n,
                                              long long p, int layout, int NT, int c_vec, int li) {
    using tt::xc;
    const long long nn = static_cast<long long>(n) * n;
    if (layout == BO_ROW_WISE && c_vec) {
        const T *ch = c + (live ? h : 0) * nn;
        // Chunk-column m of the table holds rows a <= 4m+1 (those with some
        // b >= a+2 in columns 4m..4m+3): R(m) = min(4m+2, n-2) consecutive 16-byte
        // cells in shared memory, one 16-byte piece per row (stride n) in global.
        // Lanes own column pairs (m, NT-1-m) -- equal row counts -- and stride the
        // rows by RS, so the loop is pointer increments and one asynchronous copy
        // (cp.async; measured faster than 128-bit loads + stores, 0.46 vs 0.56 ms
        // at TR-2; TMA boxes would need 128-byte aligned destinations, which the
        // packed table cannot give).
        // LPI = 8 keeps whole-row requests (lane li takes chunks li, li+8 of a
        // row): with four instances per warp the scattered column-pair requests
        // measured slower (n = 40: 0.13 -> 0.18 ms).
        if (LPI == 8 && live) {
            constexpr int LW = LPI < 16 ? LPI : 16;
            const int last_chunk = (n - 1) >> 2;
            const T *src = ch;
#pragma unroll 4
            for (int a = 0; a < n - 2; ++a, src += n) {
#pragma unroll
                for (int cc = 0; cc < 16 / LW; ++cc) {
                    const int m = ((a + 2) >> 2) + li + cc * LW;
                    if (m <= last_chunk) tt::cp_async16(Z + xc(a, m), src + 4 * m, true);
                }
            }
        } else if (live) {
            const int np = (NT + 1) >> 1;                        // column pairs
            const int RS = LPI >= 4 * np ? 4 : LPI >= 2 * np ? 2 : 1;
            if (li < np * RS) {
                const int pp = li % np, r = li / np;
#pragma unroll 1
                for (int side = 0; side < 2; ++side) {
                    const int m = side ? NT - 1 - pp : pp;
                    if (side && m == pp) break;
                    const int rows = min(4 * m + 2, n - 2);
                    T *dst = Z + xc(r, m);
                    const T *src = ch + static_cast<long long>(r) * n + 4 * m;
#pragma unroll 4
                    for (int a = r; a < rows; a += RS, dst += 4 * RS, src += static_cast<long long>(RS) * n)
                        tt::cp_async16(dst, src, true);
                }
            }
        }
        if (WAIT) tt::cp_async_wait_all();
    } else if (layout == BO_COLUMN_WISE || layout == BO_PACKED_COLUMN) {
        // Column-wise weights c[(a*n+b)*p + h] or packed c[k*p + h]: each
        // warp fetches its own two instances (on alternate lanes, so one request
        // covers 16 cells x 2 adjacent instances); the 4 warps of a CTA hold 8
        // consecutive instances, so a 32-byte sector is fetched from HBM once and
        // its other quarters hit L2.  Measured 0.72 ms at TR-2 against 0.92 ms
        // for a CTA-cooperative preload with whole-sector requests (which needs
        // two __syncthreads per instance batch and per-element index math).
        if (live) {
            const long long pl = static_cast<long long>(LPI) * p;
            for (int a = 0; a < n - 2; ++a) {
                const long long row0 = layout == BO_COLUMN_WISE ? static_cast<long long>(a) * n + a + 2
                                                                : tri_c_index(BO_PACKED_COLUMN, 0, n, 1, a, a + 2);
                const T *src = c + (row0 + li) * p + h;
                for (int b = a + 2 + li; b < n; b += LPI, src += pl) tt::cp_async4(Z + tt::xoff(a, b), src);
            }
        }
        if (WAIT) tt::cp_async_wait_all();
    } else if (live) {
        // packed row-wise or unaligned dense row-wise: 4-byte asynchronous copies
        // (a packed row is contiguous, so lanes read consecutive words)
        for (int a = 0; a < n - 2; ++a)
            for (int b = a + 2 + li; b < n; b += LPI) tt::cp_async4(Z + tt::xoff(a, b), c + tri_c_index(layout, h, n, p, a, b));
        if (WAIT) tt::cp_async_wait_all();
    }
}

// Step 1 for a whole CTA batch of column-wise weights, whole sectors
// (and of packed row-wise weights, below):
// the CTA's ninst = 8 * groups instances are consecutive and 32-byte aligned,
// so one 256-bit load brings cell (a, b) of 8 of them, and the thread writes
// the 8 values into the 8 tables (one STS each).  Warp w takes the row pairs
// (r, n-3-r), r = w, w + W, ... (n-1 cells per pair) in 32-cell pieces, so a
// warp's lanes take consecutive cells of one row: 32 consecutive b of row a
// land in distinct 16-byte bank groups (colbase(m) mod 8 runs through every
// residue over 8 consecutive m).  The per-warp path above reads 8 of every 32
// bytes it fetches and writes shared memory once per returning sector (ncu:
// ~13 wavefronts per LDGSTS, L1 at 83 %); here a 32-byte sector is one lane's
// load.  Called between two __syncthreads (the tables belong to all warps of
// the CTA here).  R loads per lane in flight: R = 1 keeps the kernel at its
// DP register count (148 at fp32 / 16 lanes); R = 2 / 4 (165 / 199 registers)
// and 4-byte cp.async copies of every cell at once measured no faster (§11).
template <typename T, int R = 1>
__device__ __forceinline__ void coop_preload_column(T *Zcta, int words, const T *__restrict__ c, long long h0,
                                                    int n, long long p, int layout, int groups) {
    struct __align__(32) V8 { T v[8]; };
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    const int npairs = (n - 1) >> 1;
    // a warp's items: its row pairs r = warp, warp + nw, ... x 32-cell pieces k x sector groups g
    const int lg = groups == 2 ? 1 : 0, lkp = n - 1 > 32 ? 1 : 0;   // (tiled kernels: n <= 64)
    const int lpp = lg + lkp;
    const int items = warp < npairs ? ((npairs - 1 - warp) / nw + 1) << lpp : 0;
    for (int i0 = 0; i0 < items; i0 += R) {
        V8 v[R];
        int off[R], grp[R];
        bool ok[R];
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const int it = i0 + u;
            const int r = warp + nw * (it >> lpp), k = (it >> lg) & lkp, g = it & lg;
            const int j = 32 * k + lane, L1 = n - 2 - r;
            const int a = j < L1 ? r : n - 3 - r;
            const int b = j < L1 ? r + 2 + j : a + 2 + (j - L1);
            ok[u] = it < items && j < n - 1 && (j < L1 || a != r);
            const bool dense = layout == BO_COLUMN_WISE || layout == BO_ROW_WISE;
            const long long e = dense ? static_cast<long long>(a) * n + b
                                      : static_cast<long long>(a) * (n - 2) - static_cast<long long>(a) * (a - 1) / 2 + (b - a - 2);
            off[u] = tt::xoff(a, b);
            grp[u] = 8 * g;
            if (ok[u]) {
                if (layout == BO_COLUMN_WISE || layout == BO_PACKED_COLUMN) {
                    v[u] = *reinterpret_cast<const V8 *>(c + e * p + h0 + 8 * g);
                } else {
                    // row-wise / packed row-wise: instance h's weights are one contiguous
                    // row of `rs` words, so the warp's 32 consecutive cells of one
                    // instance are one coalesced 128-byte request
                    const long long rs = dense ? static_cast<long long>(n) * n : static_cast<long long>(n - 1) * (n - 2) / 2;
                    const T *src = c + (h0 + 8 * g) * rs + e;
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[u].v[i] = src[i * rs];
                }
            }
        }
#pragma unroll
        for (int u = 0; u < R; ++u)
            if (ok[u]) {
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const int t = grp[u] + i;                          // table (instance) of the CTA
                    Zcta[t * words + off[u]] = v[u].v[i];
                }
            }
    }
}

// Bulk L2 prefetch of the NEXT wave of column-wise weights.  The CTAs of one
// wave (batch j of every CTA) cover the consecutive instances [w0, w0 +
// inst_stride), so each weight row (a, b) of the wave is one contiguous run of
// inst_stride * 4 bytes (14 KB for 444 CTAs x 8).  CTA k prefetches the runs of
// cells e = k, k + gridDim.x, ... with cp.async.bulk.prefetch.L2, so DRAM
// serves long sequential reads; the CTAs' own 32-byte loads then hit L2
// (without it each CTA's 32-byte sectors, 4 p bytes apart, come from a
// different DRAM row: ~2 TB/s for the copy phase alone).
template <typename T>
__device__ __forceinline__ void coop_bulk_prefetch_wave(const T *__restrict__ c, long long w0, long long span, int n,
                                                        long long p, int layout) {
    const int lane = threadIdx.x & 31;
    if ((threadIdx.x >> 5) != 0 || w0 >= p) return;
    const long long cnt = min(span, p - w0);
    const unsigned bytes = static_cast<unsigned>(cnt * sizeof(T)) & ~15u;
    if (bytes == 0) return;
    const int cells = layout == BO_COLUMN_WISE ? n * n : (n - 1) * (n - 2) / 2;
    for (int e = blockIdx.x + gridDim.x * lane; e < cells; e += 32 * gridDim.x) {
        if (layout == BO_COLUMN_WISE && (e % n) < (e / n) + 2) continue;   // not read by Algorithm OPT
        const T *src = c + static_cast<long long>(e) * p + w0;
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
    }
}

template <typename T, int LPI, bool CHORDS, bool COOP>
__global__ void __launch_bounds__(128, 1)
tri_tiled_kernel(const T *__restrict__ c, T *__restrict__ out, int16_t *__restrict__ chords, int n, long long p,
                 int layout, int NT, int c_vec, uint64_t lsched) {
    pdl_begin();
    using Op = tt::Ops<T>;
    using T4 = typename tt::V4<T>::type;
    using tt::xc;
    constexpr int IPW = 32 / LPI;                       // instances per warp
    constexpr int kLogIpw = IPW == 4 ? 2 : IPW == 2 ? 1 : 0;
    constexpr int kLogLpi = 5 - kLogIpw;
    extern __shared__ uint8_t smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // instance slot in the warp and lane within the instance: the IPW instances
    // of a warp interleave lane by lane (see table_stride)
    const int slot = lane & (IPW - 1), li = lane >> kLogIpw;
    const int words = table_stride(NT, IPW);             // per-instance table size (+ bank pad)
    const int warps_per_cta = blockDim.x >> 5;
    const int ninst = warps_per_cta * IPW;              // consecutive instances per CTA pass
    T *Z = reinterpret_cast<T *>(smem_raw) + static_cast<size_t>(warp * IPW + slot) * words;

    // zero the table once: padding cells then stay finite forever
    for (int i = li; i < words; i += LPI) Z[i] = T(0);
    __syncwarp();

    const long long inst_stride = static_cast<long long>(gridDim.x) * warps_per_cta * IPW;
    const long long nn = static_cast<long long>(n) * n;

    for (long long base = static_cast<long long>(blockIdx.x) * ninst; base < p; base += inst_stride) {
        const long long h = base + warp * IPW + slot;
        const bool live = h < p;
#ifdef BO_TRI_CLOCK
        long long clk_ = clock64();
#endif
        // ------------------------------------------------ 1. c -> upper table
#ifndef BO_TT_NOPRELOAD
        if (COOP && base + ninst <= p) {                   // CTA-uniform
            __syncthreads();                                // every table of the CTA is free
            BO_CLK_MARK(150);
            coop_preload_column<T>(reinterpret_cast<T *>(smem_raw), words, c, base, n, p, layout, ninst >> 3);
            BO_CLK_MARK(151);
            __syncthreads();
            BO_CLK_MARK(152);
            // the next wave's rows into L2 (0.492 -> 0.488 ms at TR-2 column-wise; a
            // per-sector prefetch of this CTA's next batch measured the same; prefetching 2 or 3
            // waves ahead: 0.59 / 0.62 ms)
            if (layout == BO_COLUMN_WISE || layout == BO_PACKED_COLUMN)
                coop_bulk_prefetch_wave<T>(c, base - static_cast<long long>(blockIdx.x) * ninst + inst_stride, inst_stride, n,
                                           p, layout);
        } else {
            preload_table<T, LPI>(Z, c, h, live, n, p, layout, NT, c_vec, li);
        }
#endif   // (-DBO_TT_NOPRELOAD: timing experiment only -- results are wrong)
        __syncwarp();
        BO_CLK_MARK(0);

#ifndef BO_TT_COPYONLY   // (timing experiment: preload only, results are wrong)
        // ------------------------------------------------ 2. D = 0 (diagonal tiles)
        T dg0[3] = {T(0), T(0), T(0)}, dg1[3] = {T(0), T(0), T(0)};   // diag tiles li, li + LPI (upper part)
#pragma unroll
        for (int k = 0; k < (LPI < 16 ? 2 : 1); ++k) {
            const int I = li + k * LPI;
            if (I >= NT) break;
            T *r0 = Z + xc(4 * I, I);                    // rows 4I.. of chunk-column I
            const T4 c0 = tt::ld4(r0), c1 = tt::ld4(r0 + 4);
            const T z = T(0);
            // X[a][a+1] = 0; X[0][2], X[1][3] have the single k with two zero terms
            const T t02 = Op::add(Op::add(z, z), c0.z);
            const T t13 = Op::add(Op::add(z, z), c1.w);
            const T t03 = Op::add(Op::min(Op::add(z, t13), Op::add(t02, z)), c0.w);
            tt::st4(r0, z, z, t02, t03);                 // below-diagonal words are unused
            tt::st4(r0 + 4, z, z, z, t13);
            tt::st4(r0 + 8, z, z, z, z);
            tt::st4(r0 + 12, z, z, z, z);
            T(&dg)[3] = k == 0 ? dg0 : dg1;
            dg[0] = t02; dg[1] = t03; dg[2] = t13;
        }
        __syncwarp();
        BO_CLK_MARK(1);

        // ------------------------------------------------ 3. D = 1 .. NT-1
        for (int D = 1; D < NT; ++D) {
            const int ls = static_cast<int>(lsched >> (4 * D)) & 15;     // split_log2(NT - D, D, LPI)
            // tile index in the low bits, split index q in the high bits: the 8-lane
            // phases of an LDS.128 then hold consecutive tiles of one q, whose chunk
            // addresses fall in distinct 16-byte bank groups (tools/smem_model.py:
            // 1386 -> 1124 wavefronts per instance at n = 64), and the q == 0 lanes
            // that run the fix-up are lanes 0..t-1
            const int ib = kLogLpi - ls;
            const int I0 = li & ((1 << ib) - 1), q = li >> ib;
            const int s = 1 << ls;
            if constexpr (LPI == 8) {
                // more tiles than lanes (small D, s = 1): lane li takes tiles li and
                // li + 8 together, interleaved (two independent chains per lane)
                if (NT - D > LPI) {
                    const int I1 = I0 + LPI;
                    const bool act1 = I1 < NT - D;
                    T acc0[4][4], acc1[4][4];
                    // a lane without a second tile repeats its first (result discarded)
                    tt::dense_tile2(acc0, acc1, Z, I0, act1 ? I1 : I0, D);
                    tt::finish_tile2(Z, acc0, acc1, I0, act1 ? I1 : I0, D, act1, dg0, dg1);
                    __syncwarp();
                    BO_CLK_MARK(1 + D);
                    continue;
                }
            }
            const int I = I0;
            const bool act = I < NT - D;
            const int J = I + D;
            T acc[4][4];
            // every lane starts from +inf (uniform, no divergent init branch: -1 %
            // against initialising from the first chunk)
#pragma unroll
            for (int u = 0; u < 4; ++u)
#pragma unroll
                for (int v = 0; v < 4; ++v) acc[u][v] = Op::inf();
            if (act && I + 1 + q < J) tt::dense_tile(acc, Z, I, J, I + 1 + q, s);
            BO_CLK_MARK(80 + 4 * D);
            for (int off = 1 << ib; off < LPI; off <<= 1)
#pragma unroll
                for (int u = 0; u < 4; ++u)
#pragma unroll
                    for (int v = 0; v < 4; ++v)
                        acc[u][v] = Op::min(acc[u][v], __shfl_xor_sync(0xffffffffu, acc[u][v], off * IPW));
            BO_CLK_MARK(81 + 4 * D);
            if (act && q == 0) tt::finish_tile(Z, acc, I, J, D, dg0);   // q == 0: I == li
            BO_CLK_MARK(82 + 4 * D);
            __syncwarp();
            BO_CLK_MARK(83 + 4 * D);
        }
#endif   // BO_TT_COPYONLY
        if (live && li == 0) out[h] = Z[tt::xoff(0, n - 1)];   // X[0][n-1] = Algorithm OPT's M[1,n-1]

        if constexpr (CHORDS) {
            // NEXT-1: read the optimal triangulation off the finished table.
            // Visit sub-polygons (a, b) depth first, left part first; the split of
            // (a, b) is the smallest k with X[a][k] + X[k][b] equal to the min (the
            // k Algorithm OPT's strict '<' keeps) -- recomputed here exactly,
            // with the same fp32 adds.  Each split emits (a, k) then (k, b) when
            // that part has >= 3 vertices.  Every instance has n-2 splits, so all
            // lanes of the warp run the same number of iterations.
            // The walk state is uniform over the instance's lanes (the argmin is
            // all-reduced) and lives in registers: the pending right parts (k, b)
            // are disjoint and ordered (k_last < b_last <= ... < b_first), so the
            // stack is two 64-bit masks of their starts and ends, and a pop takes
            // the lowest set bit of each.
            int a = 0, b = n - 1, t = 0;
            unsigned long long pend_k = 0, pend_b = 0;
            int16_t *oc = chords + (live ? h : 0) * 2LL * (n - 3);
            // candidate j of lane li is k = a+1+li+LPI*j: the min is xor-all-reduced,
            // then the smallest k attaining it is the lowest lane of the first j whose
            // ballot (this instance's lanes only) is non-empty
            constexpr int KJ = (64 + LPI - 1) / LPI;
            const unsigned own = IPW == 1 ? 0xffffffffu : (IPW == 2 ? 0x55555555u : 0x11111111u) << slot;
            for (int it = 0; it < n - 2; ++it) {
                T r[KJ];
                T best = Op::inf();
#pragma unroll
                for (int j = 0; j < KJ; ++j) {
                    const int k = a + 1 + li + LPI * j;
                    r[j] = k < b ? Op::add(Z[tt::xoff(a, k)], Z[tt::xoff(k, b)]) : Op::inf();
                    best = Op::min(best, r[j]);
                }
#pragma unroll
                for (int off = 1; off < LPI; off <<= 1) best = Op::min(best, __shfl_xor_sync(0xffffffffu, best, off * IPW));
                int k = n;
#pragma unroll
                for (int j = KJ - 1; j >= 0; --j) {
                    const unsigned bal = __ballot_sync(0xffffffffu, a + 1 + li + LPI * j < b && r[j] == best) & own;
                    // a select, not a branch: measured 0.832 vs 0.866 ms for TR-2 + chords (a
                    // select-only walk state machine below was slower again, 0.871; the min and
                    // the k as two redux.sync over the instance's lanes -- CREDUX, serialised per
                    // lane mask by WARPSYNC.EXCLUSIVE -- 0.887 against 0.834; warp-uniform
                    // bounds that skip empty candidate groups, butterfly rounds and whole
                    // triangle cells -- 0.982)
                    const int kj = a + 1 + ((__ffs(bal) - 1) >> (IPW == 4 ? 2 : IPW == 2 ? 1 : 0)) + LPI * j;
                    k = bal ? kj : k;
                }
                const bool left = k - a >= 2, right = b - k >= 2;
                if (li == 0 && live) {
                    if (left) *reinterpret_cast<uint32_t *>(oc + 2 * t) = static_cast<uint32_t>(a) | (static_cast<uint32_t>(k) << 16);
                    if (right) *reinterpret_cast<uint32_t *>(oc + 2 * (t + left)) = static_cast<uint32_t>(k) | (static_cast<uint32_t>(b) << 16);
                }
                t += left + right;
                if (left) {
                    if (right) pend_k |= 1ull << k, pend_b |= 1ull << b;   // (k, b) after the left part
                    b = k;
                } else if (right) {
                    a = k;
                } else if (pend_k) {                        // leaf: resume at the innermost pending part
                    a = __ffsll(static_cast<long long>(pend_k)) - 1;
                    b = __ffsll(static_cast<long long>(pend_b)) - 1;
                    pend_k &= pend_k - 1;
                    pend_b &= pend_b - 1;
                }
            }
        }
        __syncwarp();
    }
}

int tiled_supported(int64_t n) { return n >= 3 && n <= 64; }

#ifdef BO_TRI_CLOCK
}  // namespace bo
extern "C" int bulk_debug_tri_clock(unsigned long long *host160, int reset) {
    if (reset) {
        unsigned long long z[160] = {};
        return cudaMemcpyToSymbol(bo::g_tri_clock, z, sizeof z) == cudaSuccess ? 0 : -3;
    }
    return cudaMemcpyFromSymbol(host160, bo::g_tri_clock, 160 * sizeof(unsigned long long)) == cudaSuccess ? 0 : -3;
}
namespace bo {
#endif

template <typename T, int LPI, bool CHORDS>
static int launch_tiled_t(const void *c, void *out, int16_t *chords, int64_t n, int64_t p, int layout,
                          cudaStream_t st) {
    const int NT = static_cast<int>((n + 3) / 4);
    constexpr int IPW = 32 / LPI;
    const size_t per_inst = static_cast<size_t>(table_stride(NT, IPW)) * sizeof(T);
    const bool column = layout == BO_COLUMN_WISE || layout == BO_PACKED_COLUMN;
    // warps per CTA: the W in 1..4 that keeps the most warps resident per SM
    // (shared memory is the limit: 227 KB, 1 KB reserved per CTA)
    int W = 1, best = 0;
    for (int w = 1; w <= 4; ++w) {
        const size_t per_cta = w * IPW * per_inst + 1024;
        const int resident = static_cast<int>((227 * 1024) / per_cta) * w;
        // (column-wise and packed row-wise weights: prefer 4 warps, 8+ instances per batch for the
        // cooperative preload)
        const bool prefer4 = column || layout == BO_PACKED_ROW;
        if (resident > best || (prefer4 && resident == best)) best = resident, W = w;
    }
    const size_t smem = W * IPW * per_inst;
    const long long per_cta = static_cast<long long>(W) * IPW;
    const int c_vec = (n % 4 == 0) && aligned16(c);
    // whole-sector CTA preload of column-wise weights (8 or 16 consecutive,
    // 32-byte aligned instances per CTA batch): a kernel of its own, so the
    // per-warp kernels keep their register allocation
    bool coop = false;
#ifndef BO_TT_NOCOOP
    // (packed row-wise too: scalar loads, no alignment needed -- TR-2 packed 0.620 -> 0.499 ms; dense
    // row-wise stays per-warp: its 16-byte cp.async rows measured 0.371 against 0.512 ms cooperative)
    coop = (column && p % 8 == 0 && (reinterpret_cast<uintptr_t>(c) & 31u) == 0) || layout == BO_PACKED_ROW;
    coop = coop && (per_cta == 8 || per_cta == 16);
#endif
    const auto kern = coop ? &tri_tiled_kernel<T, LPI, CHORDS, true> : &tri_tiled_kernel<T, LPI, CHORDS, false>;
    const bool attr = ensure_dyn_smem(reinterpret_cast<const void *>(kern), 227 * 1024);
    if (!attr) return fail(BO_ECUDA, "tiled: cannot set dynamic smem");
    int per_sm = max_blocks_per_sm(reinterpret_cast<const void *>(kern), W * 32, smem);
    per_sm = std::max(per_sm, 1);
    const long long blocks = std::min<long long>((p + per_cta - 1) / per_cta,
                                                 static_cast<long long>(per_sm) * num_sms());
    launch(kern, static_cast<unsigned>(blocks), W * 32, smem, st,
        static_cast<const T *>(c), static_cast<T *>(out), chords, static_cast<int>(n), p, layout, NT, c_vec,
        split_schedule(NT, LPI));
    return after_launch("tri_tiled_kernel");
}

// lpi: lanes per instance (BO_TRI_TILED = 32, BO_TRI_TILED_HALF = 16, BO_TRI_TILED_QUARTER = 8)
int launch_tri_tiled(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout, int lpi,
                     cudaStream_t st) {
    if (dtype == BO_F32)
        return lpi == 16 ? launch_tiled_t<float, 16, false>(c, out, nullptr, n, p, layout, st)
               : lpi == 8 ? launch_tiled_t<float, 8, false>(c, out, nullptr, n, p, layout, st)
                          : launch_tiled_t<float, 32, false>(c, out, nullptr, n, p, layout, st);
    return lpi == 16 ? launch_tiled_t<int32_t, 16, false>(c, out, nullptr, n, p, layout, st)
           : lpi == 8 ? launch_tiled_t<int32_t, 8, false>(c, out, nullptr, n, p, layout, st)
                      : launch_tiled_t<int32_t, 32, false>(c, out, nullptr, n, p, layout, st);
}

// NEXT-1: values and the chords of an optimal triangulation (16 lanes per instance)
int launch_tri_chords(const void *c, void *out, int16_t *chords, int64_t n, int64_t p, int dtype, int layout,
                      cudaStream_t st) {
    if (dtype == BO_F32) return launch_tiled_t<float, 16, true>(c, out, chords, n, p, layout, st);
    return launch_tiled_t<int32_t, 16, true>(c, out, chords, n, p, layout, st);
}

// ---------------------------------------------------------------------------
// TILED_GLOBAL (NEXT-2, large polygons, e.g. the paper's 512-gons):
// the same blocked algorithm with one CTA per instance and the chunk-column
// table in a global workspace slot per CTA (grid = #SMs, so the working set
// stays L2-resident: 530 KB x 148 = 78 MB at n = 512).  __syncthreads orders
// the tile-diagonals; a tile's split lanes stay inside one warp (s <= 32).
// ---------------------------------------------------------------------------
__device__ __forceinline__ int split_log2_cta(int t, int D, int threads) {
    int ls = 0;
    while ((2 << ls) * t <= threads && (1 << ls) < D - 1 && (2 << ls) <= 32) ++ls;
    return ls;
}

template <typename T>
__global__ void __launch_bounds__(512, 1)
tri_tiled_global_kernel(const T *__restrict__ c, T *__restrict__ out, T *ws, int n, long long p, int layout, int NT,
                        int c_vec) {
    pdl_begin();
    using Op = tt::Ops<T>;
    using T4 = typename tt::V4<T>::type;
    using tt::xc;
    const long long words = 4LL * tt::colbase(NT);
    T *Z = ws + static_cast<long long>(blockIdx.x) * words;
    const int tid = threadIdx.x, nthr = blockDim.x;
    const long long nn = static_cast<long long>(n) * n;
    for (long long i = tid; i < words; i += nthr) Z[i] = T(0);      // padding stays finite
    for (long long h = blockIdx.x; h < p; h += gridDim.x) {
        __syncthreads();
        // 1. weights b >= a+2 -> upper table
        if (layout == BO_ROW_WISE && c_vec) {
            const T4 *src = reinterpret_cast<const T4 *>(c + h * nn);
            for (int idx = tid; idx < (n - 2) * NT; idx += nthr) {
                const int a = idx / NT, m = idx - a * NT;
                if (m >= ((a + 2) >> 2)) *reinterpret_cast<T4 *>(Z + xc(a, m)) = __ldg(src + static_cast<long long>(a) * (n / 4) + m);
            }
        } else {
            for (int a = 0; a < n - 2; ++a)
                for (int b = a + 2 + tid; b < n; b += nthr) Z[tt::xoff(a, b)] = __ldg(c + tri_c_index(layout, h, n, p, a, b));
        }
        __syncthreads();
        // 2. D = 0
        for (int I = tid; I < NT; I += nthr) {
            T *r0 = Z + xc(4 * I, I);
            const T4 c0 = tt::ld4(r0), c1 = tt::ld4(r0 + 4);
            const T z = T(0);
            const T t02 = Op::add(Op::add(z, z), c0.z);
            const T t13 = Op::add(Op::add(z, z), c1.w);
            const T t03 = Op::add(Op::min(Op::add(z, t13), Op::add(t02, z)), c0.w);
            tt::st4(r0, z, z, t02, t03);
            tt::st4(r0 + 4, z, z, z, t13);
            tt::st4(r0 + 8, z, z, z, z);
            tt::st4(r0 + 12, z, z, z, z);
        }
        __syncthreads();
        // 3. tile-diagonals
        for (int D = 1; D < NT; ++D) {
            const int t = NT - D;
            const int ls = split_log2_cta(t, D, nthr);
            const int s = 1 << ls;
            for (int base = 0; base < t * s; base += nthr) {       // more tiles than threads: loop
                const int slot = base + tid;
                const int I = slot >> ls, q = slot & (s - 1);
                const bool act = I < t;
                const int J = I + D;
                T acc[4][4];
#pragma unroll
                for (int u = 0; u < 4; ++u)
#pragma unroll
                    for (int v = 0; v < 4; ++v) acc[u][v] = Op::inf();
                if (act) {
                    for (int m = I + 1 + q; m < J; m += s) {
                        const T *pa = Z + xc(4 * I, m), *pb = Z + xc(4 * m, J);
                        T4 A[4], B[4];
#pragma unroll
                        for (int u = 0; u < 4; ++u) A[u] = tt::ld4(pa + 4 * u), B[u] = tt::ld4(pb + 4 * u);
                        tt::minplus_chunk(acc, A, B);
                    }
                }
                for (int off = 1; off < s; off <<= 1)
#pragma unroll
                    for (int u = 0; u < 4; ++u)
#pragma unroll
                        for (int v = 0; v < 4; ++v)
                            acc[u][v] = Op::min(acc[u][v], __shfl_xor_sync(0xffffffffu, acc[u][v], off));
                if (act && q == 0) {
                    T *ta = Z + xc(4 * I, I), *tb = Z + xc(4 * J, J), *tc = Z + xc(4 * I, J);
                    T A[4][4], Bd[4][4], C[4][4];
#pragma unroll
                    for (int r = 0; r < 4; ++r) {
                        const T4 x = tt::ld4(ta + 4 * r), y = tt::ld4(tb + 4 * r), w = tt::ld4(tc + 4 * r);
                        A[r][0] = x.x; A[r][1] = x.y; A[r][2] = x.z; A[r][3] = x.w;
                        Bd[r][0] = y.x; Bd[r][1] = y.y; Bd[r][2] = y.z; Bd[r][3] = y.w;
                        C[r][0] = w.x; C[r][1] = w.y; C[r][2] = w.z; C[r][3] = w.w;
                    }
                    T tt_[4][4];
                    tt::fixup(tt_, acc, A, Bd, C, D == 1);
#pragma unroll
                    for (int u = 0; u < 4; ++u) tt::st4(tc + 4 * u, tt_[u][0], tt_[u][1], tt_[u][2], tt_[u][3]);
                }
            }
            __syncthreads();
        }
        if (tid == 0) out[h] = Z[tt::xoff(0, n - 1)];
    }
}

int tiled_global_threads(int64_t n) { return n >= 256 ? 512 : 256; }

size_t tiled_global_workspace(int64_t n, int64_t p) {
    const int NT = static_cast<int>((n + 3) / 4);
    const long long grid = std::min<long long>(p, num_sms());
    return static_cast<size_t>(grid) * 4 * tt::colbase(NT) * 4;
}

int launch_tri_tiled_global(const void *c, void *out, void *ws, int64_t n, int64_t p, int dtype, int layout,
                            cudaStream_t st) {
    // the kernel moves table rows with 16-byte vector loads and stores
    if ((reinterpret_cast<uintptr_t>(ws) & 15u) != 0) return fail(BO_EINVAL, "TILED_GLOBAL: workspace must be 16-byte aligned");
    const int NT = static_cast<int>((n + 3) / 4);
    const long long grid = std::min<long long>(p, num_sms());
    const int threads = tiled_global_threads(n);
    const int c_vec = (n % 4 == 0) && aligned16(c);
    if (dtype == BO_F32)
        launch(tri_tiled_global_kernel<float>, static_cast<unsigned>(grid), threads, 0, st, 
            static_cast<const float *>(c), static_cast<float *>(out), static_cast<float *>(ws), static_cast<int>(n), p,
            layout, NT, c_vec);
    else
        launch(tri_tiled_global_kernel<int32_t>, static_cast<unsigned>(grid), threads, 0, st, 
            static_cast<const int32_t *>(c), static_cast<int32_t *>(out), static_cast<int32_t *>(ws),
            static_cast<int>(n), p, layout, NT, c_vec);
    return after_launch("tri_tiled_global_kernel");
}

}  // namespace bo
