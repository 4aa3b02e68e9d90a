// prefix.cu -- bulk inclusive prefix sums (Algorithm Prefix-sums, P:95-102;
// Parallel Algorithm Prefix-sums).
//
// Every variant except WARPSCAN keeps the paper's left-to-right order
// r <- r + b[i] per instance, so fp32 results are bit-identical to the
// sequential algorithm.  int32 adds wrap mod 2^32.
//
//  ACROSS     column-wise [n][p]: a TMA ring of [64 rows x 128
//             instances] boxes, thread t scans column t in shared memory
//             (ps_across_tma); or, for short columns / unaligned data, a
//             thread owns 4 adjacent instances, one 128-bit coalesced
//             load/store per row i, U rows of loads in flight (the addresses
//             are input-independent -- obliviousness, P:91 -- so they can be
//             issued far ahead of the adds).
//  FUSED_ROW  row-wise [p][n]: TMA brings [128 instances x 32 elems]
//             boxes (128B swizzle) into a smem ring; thread t scans instance t
//             sequentially out of smem (conflict-free 128-bit reads), writes
//             in place, TMA stores the box.  The row->column transpose happens
//             on chip: HBM traffic = 2*n*p*4 bytes, same as column-wise.
//  WARPSCAN   row-wise: warp per instance, shuffle scan (fp32 reassociated).
//  NAIVE      the paper's kernel: one thread per instance, scalar accesses in
//             the given arrangement -- the prior-art baseline.
#include "common.cuh"

namespace bo {

int launch_transpose(const void *src, void *dst, int64_t rows, int64_t cols, cudaStream_t st);

template <typename T>
__device__ __forceinline__ T bits_as(uint32_t u) {
    if constexpr (sizeof(T) == 4 && std::is_same<T, float>::value) return __uint_as_float(u);
    else return static_cast<T>(u);
}
template <typename T>
__device__ __forceinline__ uint32_t as_bits(T v) {
    if constexpr (std::is_same<T, float>::value) return __float_as_uint(v);
    else return static_cast<uint32_t>(v);
}

// ------------------------------------------------------------------ ACROSS
template <typename T, int U>
__global__ void __launch_bounds__(256)
ps_across_vec4(const T *src, T *dst, long long n, long long p4) {
    pdl_begin();
    const long long g = blockIdx.x * 256LL + threadIdx.x;
    if (g >= p4) return;
    const uint4 *s = reinterpret_cast<const uint4 *>(src) + g;
    uint4 *d = reinterpret_cast<uint4 *>(dst) + g;
    T r0 = T(0), r1 = T(0), r2 = T(0), r3 = T(0);
    long long i = 0;
    for (; i + U <= n; i += U) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = __ldcs(s + (i + u) * p4);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            r0 = add_wrap(r0, bits_as<T>(v[u].x));
            r1 = add_wrap(r1, bits_as<T>(v[u].y));
            r2 = add_wrap(r2, bits_as<T>(v[u].z));
            r3 = add_wrap(r3, bits_as<T>(v[u].w));
            __stcs(d + (i + u) * p4, make_uint4(as_bits(r0), as_bits(r1), as_bits(r2), as_bits(r3)));
        }
    }
    for (; i < n; ++i) {
        const uint4 v = __ldcs(s + i * p4);
        r0 = add_wrap(r0, bits_as<T>(v.x));
        r1 = add_wrap(r1, bits_as<T>(v.y));
        r2 = add_wrap(r2, bits_as<T>(v.z));
        r3 = add_wrap(r3, bits_as<T>(v.w));
        __stcs(d + i * p4, make_uint4(as_bits(r0), as_bits(r1), as_bits(r2), as_bits(r3)));
    }
}

template <typename T, int U>
__global__ void __launch_bounds__(256)
ps_across_scalar(const T *src, T *dst, long long n, long long p) {
    pdl_begin();
    const long long j = blockIdx.x * 256LL + threadIdx.x;
    if (j >= p) return;
    T r = T(0);
    long long i = 0;
    for (; i + U <= n; i += U) {
        T v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = src[(i + u) * p + j];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            r = add_wrap(r, v[u]);
            dst[(i + u) * p + j] = r;
        }
    }
    for (; i < n; ++i) {
        r = add_wrap(r, src[i * p + j]);
        dst[i * p + j] = r;
    }
}

// --------------------------------------------------------------- FUSED_ROW
namespace fr {
// INST instances per tile = threads per CTA: 128 normally, 32 when p is so
// small that 128-instance tiles would leave SMs idle (p < 2 * SMs * 128).
constexpr int kElems = 32;                 // elements per chunk (128 B rows, swizzle 128B)
template <int INST> struct Cfg {
#ifndef BO_FR_STAGES
#define BO_FR_STAGES 8      // measured: 1 CTA/SM with a 7-8 deep ring beats 2 CTAs x 6 (99.3 % vs 96.0 % of HBM)
#endif
    // 32-instance tiles serve small p.  Chunks (TMA boxes) per ring stage: a stage's
    // scan, barrier and stores are one dependent round of the CTA, so with 4 KiB
    // boxes several chunks per stage keep that fixed cost off each box.  Measured
    // (stages x chunks): 3 x 4 against 8 x 1 -- n = 32K p = 8K 0.477 vs 0.554 ms,
    // n = 4096 p = 8192 65 vs 73 us, n = 1024 p = 4096 18.2 vs 20.9 us, p = 32768 48.7
    // vs 50.5 us, p = 16384 23.9 vs 23.6 us; 4 x 4 and 6 x 4 lose at p = 16384 (34 us:
    // fewer CTAs per SM than tiles), a 24 x 1 ring loses everywhere.  After the scan
    // was register-staged (late round 2) the ring depth matters again: 6 x 2 (the same
    // 48 KB) against 3 x 4 -- n = 32K p = 8K 0.369 vs 0.403 ms, n = 4096 p = 8192 48.2 vs
    // 54.6 us, n = 1024 p = 16384 / 32768 22.1 / 45.6 vs 22.2 / 46.2 us, n = 1024
    // p = 4096 13.3 vs 12.9 us; 4 x 4 loses at p = 16384 (26.9 us).
#ifndef BO_FR_STAGES32
#define BO_FR_STAGES32 6
#endif
#ifndef BO_FR_CPS32
#define BO_FR_CPS32 2
#endif
    static constexpr int kStages = INST == 128 ? BO_FR_STAGES : BO_FR_STAGES32;
    static constexpr int kCps = INST == 128 ? 1 : BO_FR_CPS32;
    static constexpr uint32_t kBoxBytes = INST * kElems * 4;   // 16 KiB / 4 KiB
    static constexpr uint32_t kStageBytes = kCps * kBoxBytes;
    static constexpr size_t kSmem = 1024 + kStages * kStageBytes + kStages * 20;
};
}  // namespace fr

__device__ WorkSlot g_fr_slots[kWorkSlots];

template <typename T, int kInst>
__global__ void __launch_bounds__(kInst)
ps_fused_row_tma(const __grid_constant__ CUtensorMap src_map, const __grid_constant__ CUtensorMap dst_map,
                 long long ntiles, int nchunks, int slot) {
    pdl_begin();
    using fr::kElems;
    constexpr int kStages = fr::Cfg<kInst>::kStages;
    constexpr int kCps = fr::Cfg<kInst>::kCps;
    constexpr uint32_t kBoxBytes = fr::Cfg<kInst>::kBoxBytes;
    constexpr uint32_t kStageBytes = fr::Cfg<kInst>::kStageBytes;
    extern __shared__ uint8_t smem_raw[];
    uint8_t *buf = smem_align<1024>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(buf + kStages * kStageBytes);
    int *stage_tile = reinterpret_cast<int *>(full + kStages);    // tile of each ring slot, -1 = end
    int *stage_chunk = stage_tile + kStages;                      // its first chunk
    int *stage_cnt = stage_chunk + kStages;                       // and how many (<= kCps, one tile)
    WorkSlot *ws = slot >= 0 ? &g_fr_slots[slot] : nullptr;
    const int tid = threadIdx.x;

    if (tid == 0) {
        prefetch_tmap(&src_map);
        prefetch_tmap(&dst_map);
        for (int s = 0; s < kStages; ++s) mbar_init(&full[s], 1);
        fence_barrier_init();
    }
    __syncthreads();

    // producer state (thread 0 only): next (tile, chunk) to load
    long long prod_tile = blockIdx.x;
    int prod_chunk = 0;
    bool prod_done = false;
    auto issue = [&](int s) {
        if (prod_chunk == nchunks) {
            prod_tile = claim_tile(ws, prod_tile);
            prod_chunk = 0;
        }
        if (prod_tile >= ntiles) {
            stage_tile[s] = -1;
            prod_done = true;
            mbar_arrive(&full[s]);
            return;
        }
        stage_tile[s] = static_cast<int>(prod_tile);
        stage_chunk[s] = prod_chunk;
        if constexpr (kCps == 1) {
            mbar_arrive_expect_tx(&full[s], kBoxBytes);
            tma_load_2d(buf + s * kStageBytes, &src_map, prod_chunk * kElems, static_cast<int>(prod_tile * kInst),
                        &full[s]);
            ++prod_chunk;
        } else {
            const int cnt = min(kCps, nchunks - prod_chunk);
            stage_cnt[s] = cnt;
            mbar_arrive_expect_tx(&full[s], cnt * kBoxBytes);
            for (int b = 0; b < cnt; ++b)
                tma_load_2d(buf + s * kStageBytes + b * kBoxBytes, &src_map, (prod_chunk + b) * kElems,
                            static_cast<int>(prod_tile * kInst), &full[s]);
            prod_chunk += cnt;
        }
    };
    if (tid == 0)
        for (int s = 0; s < kStages - 1 && !prod_done; ++s) issue(s);

    T r = T(0);
    for (long long i = 0;; ++i) {
        const int s = static_cast<int>(i % kStages);
        mbar_wait(&full[s], static_cast<uint32_t>((i / kStages) & 1));
        const int tile = stage_tile[s];
        if (tile < 0) break;
        const int chunk = stage_chunk[s];
        const int cnt = kCps == 1 ? 1 : stage_cnt[s];
        if (chunk == 0) r = T(0);                       // new tile: r_j <- 0
        // a box's 8 row pieces read into registers before the dependent chain, the next
        // box's while this one is scanned (the swizzled addresses defeat the compiler's
        // alias analysis, so in-place load / add / store pieces serialise on each other):
        // with shared-space addressing, n = 32K p = 8K 0.468 -> 0.403 ms, n = 1024 p = 4096
        // 17.9 -> 12.9 us, n = 4096 p = 8192 63 -> 55 us; PS-2 1.320 -> 1.318 ms
        uint4 cur[kElems / 4], nxt[kElems / 4];
#pragma unroll
        for (int k = 0; k < kElems / 4; ++k)
            cur[k] = *reinterpret_cast<const uint4 *>(buf + s * kStageBytes + swz128(tid, k));
#pragma unroll
        for (int b = 0; b < kCps; ++b) {
            if (kCps > 1 && b >= cnt) break;
            uint8_t *box = buf + s * kStageBytes + b * kBoxBytes;
            if (b + 1 < kCps && b + 1 < cnt) {
#pragma unroll
                for (int k = 0; k < kElems / 4; ++k)
                    nxt[k] = *reinterpret_cast<const uint4 *>(box + kBoxBytes + swz128(tid, k));
            }
#pragma unroll
            for (int k = 0; k < kElems / 4; ++k) {
                uint4 v = cur[k];
                r = add_wrap(r, bits_as<T>(v.x)); v.x = as_bits(r);   // r <- r + b[i]; b[i] <- r
                r = add_wrap(r, bits_as<T>(v.y)); v.y = as_bits(r);
                r = add_wrap(r, bits_as<T>(v.z)); v.z = as_bits(r);
                r = add_wrap(r, bits_as<T>(v.w)); v.w = as_bits(r);
                cur[k] = v;
            }
#pragma unroll
            for (int k = 0; k < kElems / 4; ++k) *reinterpret_cast<uint4 *>(box + swz128(tid, k)) = cur[k];
#pragma unroll
            for (int k = 0; k < kElems / 4; ++k) cur[k] = nxt[k];
        }
        fence_proxy_async_smem();
        __syncthreads();
        if (tid == 0) {
#pragma unroll
            for (int b = 0; b < kCps; ++b) {
                if (kCps > 1 && b >= cnt) break;
                tma_store_2d(&dst_map, buf + s * kStageBytes + b * kBoxBytes, (chunk + b) * kElems, tile * kInst);
            }
            bulk_commit();
            bulk_wait_read<1>();                       // stage i-1's stores no longer read it
            if (!prod_done) issue(static_cast<int>((i + kStages - 1) % kStages));
        }
    }
    if (tid == 0) {
        bulk_wait<0>();
        retire_cta(ws);
    }
}

// ACROSS on column-wise [n][p] through the same TMA ring: a tile is a block
// of kInst consecutive instances (columns), walked down in chunks of kElems
// rows; a box [kElems rows x kInst instances] lands unswizzled, so thread t
// scans column t with conflict-free 32-bit shared accesses, in place, and the
// box is stored back by TMA.  No transposition is involved: this is the
// paper's column-wise bulk order with HBM streamed by TMA.
namespace ac {
#ifndef BO_AC_ROWS
#define BO_AC_ROWS 64
#endif
#ifndef BO_AC_STAGES
#define BO_AC_STAGES 4
#endif
// measured at PS-2 column-wise: 64-row boxes x 4 stages (2 CTAs/SM) 1.349 ms,
// 32 x 8 1.356, 32 x 4 1.360, 64 x 3 1.356, 16 x 8 1.360
constexpr int kElems = BO_AC_ROWS;          // rows per box
constexpr int kStages = BO_AC_STAGES;
// 32-instance blocks, ring depth with shared-space scan accesses (late round 2; the
// round-2 generic pointer had 12): 4 / 6 / 8 / 12 / 24 stages -- n = 32K p = 8K 0.392 /
// 0.358 / 0.401 / 0.425 / 0.535 ms, n = 4096 p = 8192 52.0 / 43.9 / 49.7 / 53.1 / 72.2 us
// (generic, 12: 0.383 ms, 52.4 us), n = 1024 p = 16384 22.1 / 22.7 / 24.4 / 23.6 us (29.4)
#ifndef BO_AC_STAGES32
#define BO_AC_STAGES32 6
#endif
template <int INST> struct Cfg {
    // 32-instance column blocks (small p, long columns): a deeper ring per CTA
    static constexpr int kStages = INST == 128 ? ac::kStages : BO_AC_STAGES32;
    static constexpr uint32_t kBoxBytes = INST * kElems * 4;
    static constexpr size_t kSmem = 1024 + kStages * kBoxBytes + kStages * 16;
};
}  // namespace ac

template <typename T, int kInst>
__global__ void __launch_bounds__(kInst)
ps_across_tma(const __grid_constant__ CUtensorMap src_map, const __grid_constant__ CUtensorMap dst_map,
              long long ntiles, int nchunks, int slot) {
    pdl_begin();
    using ac::kElems;
    constexpr int kStages = ac::Cfg<kInst>::kStages;
    constexpr uint32_t kBoxBytes = ac::Cfg<kInst>::kBoxBytes;
    extern __shared__ uint8_t smem_raw[];
    uint8_t *buf = smem_align<1024>(smem_raw);
    uint64_t *full = reinterpret_cast<uint64_t *>(buf + kStages * kBoxBytes);
    int *stage_tile = reinterpret_cast<int *>(full + kStages);
    int *stage_chunk = stage_tile + kStages;
    WorkSlot *ws = slot >= 0 ? &g_fr_slots[slot] : nullptr;
    const int tid = threadIdx.x;
    if (tid == 0) {
        prefetch_tmap(&src_map);
        prefetch_tmap(&dst_map);
        for (int s = 0; s < kStages; ++s) mbar_init(&full[s], 1);
        fence_barrier_init();
    }
    __syncthreads();
    long long prod_tile = blockIdx.x;
    int prod_chunk = 0;
    bool prod_done = false;
    auto issue = [&](int s) {
        if (prod_chunk == nchunks) {
            prod_tile = claim_tile(ws, prod_tile);
            prod_chunk = 0;
        }
        if (prod_tile >= ntiles) {
            stage_tile[s] = -1;
            prod_done = true;
            mbar_arrive(&full[s]);
            return;
        }
        stage_tile[s] = static_cast<int>(prod_tile);
        stage_chunk[s] = prod_chunk;
        mbar_arrive_expect_tx(&full[s], kBoxBytes);
        tma_load_2d(buf + s * kBoxBytes, &src_map, static_cast<int>(prod_tile * kInst), prod_chunk * kElems,
                    &full[s]);
        ++prod_chunk;
    };
    if (tid == 0)
        for (int s = 0; s < kStages - 1 && !prod_done; ++s) issue(s);
    T r = T(0);
    for (long long i = 0;; ++i) {
        const int s = static_cast<int>(i % kStages);
        mbar_wait(&full[s], static_cast<uint32_t>((i / kStages) & 1));
        const int tile = stage_tile[s];
        if (tile < 0) break;
        const int chunk = stage_chunk[s];
        if (chunk == 0) r = T(0);                       // new column block: r_j <- 0
        uint32_t *box = reinterpret_cast<uint32_t *>(buf + s * kBoxBytes) + tid;
#pragma unroll
        for (int e = 0; e < kElems; ++e) {              // r <- r + b[i]; b[i] <- r
            r = add_wrap(r, bits_as<T>(box[e * kInst]));
            box[e * kInst] = as_bits(r);
        }
        fence_proxy_async_smem();
        __syncthreads();
        if (tid == 0) {
            tma_store_2d(&dst_map, buf + s * kBoxBytes, tile * kInst, chunk * kElems);
            bulk_commit();
            bulk_wait_read<1>();
            if (!prod_done) issue(static_cast<int>((i + kStages - 1) % kStages));
        }
    }
    if (tid == 0) {
        bulk_wait<0>();
        retire_cta(ws);
    }
}

// Fallback for any n / alignment: coalesced warp loads into a padded tile.
template <typename T>
__global__ void __launch_bounds__(128)
ps_fused_row_smem(const T *src, T *dst, long long n, long long p) {
    pdl_begin();
    __shared__ T tile[128][33];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    for (long long t0 = blockIdx.x * 128LL; t0 < p; t0 += 128LL * gridDim.x) {
        T r = T(0);
        for (long long c0 = 0; c0 < n; c0 += 32) {
            for (int row = warp; row < 128; row += 4) {
                const long long h = t0 + row, c = c0 + lane;
                tile[row][lane] = (h < p && c < n) ? src[h * n + c] : T(0);
            }
            __syncthreads();
#pragma unroll 8
            for (int e = 0; e < 32; ++e) {
                r = add_wrap(r, tile[tid][e]);
                tile[tid][e] = r;
            }
            __syncthreads();
            for (int row = warp; row < 128; row += 4) {
                const long long h = t0 + row, c = c0 + lane;
                if (h < p && c < n) dst[h * n + c] = tile[row][lane];
            }
            __syncthreads();
        }
    }
}

// ---------------------------------------------------------------- WARPSCAN
template <typename T>
__device__ __forceinline__ T warp_incl_scan(T x, int lane) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x = add_wrap(y, x);
    }
    return x;
}

template <typename T, bool kVec>
__global__ void __launch_bounds__(256)
ps_warpscan(const T *src, T *dst, long long n, long long p) {
    pdl_begin();
    const int lane = threadIdx.x & 31;
    const long long warps = (static_cast<long long>(gridDim.x) * blockDim.x) >> 5;
    for (long long h = (blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x) >> 5; h < p;
         h += warps) {
        const T *s = src + h * n;
        T *d = dst + h * n;
        T carry = T(0);
        if (kVec) {
            for (long long c = 0; c < n; c += 128) {
                const long long idx = c + lane * 4;
                uint4 v = idx < n ? __ldcs(reinterpret_cast<const uint4 *>(s + idx)) : make_uint4(0, 0, 0, 0);
                T a = bits_as<T>(v.x), b = bits_as<T>(v.y), e = bits_as<T>(v.z), f = bits_as<T>(v.w);
                b = add_wrap(a, b);
                e = add_wrap(b, e);
                f = add_wrap(e, f);
                const T incl = warp_incl_scan(f, lane);
                T excl = __shfl_up_sync(0xffffffffu, incl, 1);
                excl = lane == 0 ? carry : add_wrap(carry, excl);
                if (idx < n)
                    __stcs(reinterpret_cast<uint4 *>(d + idx),
                           make_uint4(as_bits(add_wrap(excl, a)), as_bits(add_wrap(excl, b)),
                                      as_bits(add_wrap(excl, e)), as_bits(add_wrap(excl, f))));
                carry = add_wrap(carry, __shfl_sync(0xffffffffu, incl, 31));
            }
        } else {
            for (long long c = 0; c < n; c += 32) {
                const long long idx = c + lane;
                const T v = idx < n ? s[idx] : T(0);
                const T incl = warp_incl_scan(v, lane);
                if (idx < n) d[idx] = add_wrap(carry, incl);
                carry = add_wrap(carry, __shfl_sync(0xffffffffu, incl, 31));
            }
        }
    }
}

// ------------------------------------------------------------------- NAIVE
// Parallel Algorithm Prefix-sums exactly as printed: thread T(j)
// keeps r_j and walks its array with one 32-bit access per step.
template <typename T>
__global__ void __launch_bounds__(64)
ps_naive(const T *src, T *dst, long long n, long long p, int layout) {
    pdl_begin();
    const long long j = blockIdx.x * 64LL + threadIdx.x;
    if (j >= p) return;
    T r = T(0);
    for (long long i = 0; i < n; ++i) {
        const long long a = layout == BO_ROW_WISE ? j * n + i : i * p + j;
        r = add_wrap(r, src[a]);
        dst[a] = r;
    }
}

// ------------------------------------------------------------------- host
bool fused_tma_ok(const void *src, const void *dst, int64_t n, int64_t p) {
    return aligned16(src) && aligned16(dst) && n % 4 == 0 && n < (int64_t(1) << 31) &&
           p < (int64_t(1) << 31);
}

int resolve_prefix_variant(int64_t n, int64_t p, int dtype, int layout, int variant, const void *src,
                           const void *dst) {
    (void)n; (void)src; (void)dst;
    if (variant != BO_AUTO) return variant;
    if (layout == BO_COLUMN_WISE) return BO_PS_ACROSS;
    // int32 addition is associative mod 2^32, so the warp-scan is bit-exact too;
    // it wins when there are too few instances to fill the GPU with 128-instance
    // TMA tiles (measured: PS-1, n=32 p=1024, 6.2 vs 8.2 us).  fp32 keeps the
    // sequential order (FUSED_ROW) so results stay bit-identical to P:100.
    if (dtype == BO_I32 && p < 2LL * 128 * num_sms()) return BO_PS_WARPSCAN;
    return BO_PS_FUSED_ROW;
}

template <typename T, int INST>
static int launch_across_tma(const T *src, T *dst, int64_t n, int64_t p, cudaStream_t st) {
    using C = ac::Cfg<INST>;
    CUtensorMap smap, dmap;
    if (!make_tmap_2d(&smap, src, n, p, ac::kElems, INST, CU_TENSOR_MAP_SWIZZLE_NONE) ||
        !make_tmap_2d(&dmap, dst, n, p, ac::kElems, INST, CU_TENSOR_MAP_SWIZZLE_NONE))
        return fail(BO_ECUDA, "prefix across: cuTensorMapEncodeTiled failed");
    const bool attr = ensure_dyn_smem(reinterpret_cast<const void *>(&ps_across_tma<T, INST>), static_cast<int>(C::kSmem));
    if (!attr) return fail(BO_ECUDA, "prefix across: cannot set dynamic smem");
    const long long ntiles = (p + INST - 1) / INST;
    const int nchunks = static_cast<int>((n + ac::kElems - 1) / ac::kElems);
    int per_sm = 1;
    per_sm = max_blocks_per_sm(reinterpret_cast<const void *>(&ps_across_tma<T, INST>), INST, C::kSmem);
    const long long grid = std::min<long long>(ntiles, static_cast<long long>(std::max(per_sm, 1)) * num_sms());
    const int slot = work_slot_for(st);
    launch(ps_across_tma<T, INST>, static_cast<unsigned>(grid), INST, C::kSmem, st, smap, dmap, ntiles, nchunks, slot);
    return after_launch("ps_across_tma");
}

#ifndef BO_ACROSS_TMA
#define BO_ACROSS_TMA 1
#endif
template <typename T>
static int launch_across(const T *src, T *dst, int64_t n, int64_t p, cudaStream_t st) {
    // TMA ring when the rows are 16-byte aligned, there are enough 128-instance
    // column blocks to give every SM work, and a block has several row chunks
    // (measured: PS-2 column-wise 1.356 vs 1.384 ms; n = 32, p = 2^22: 0.188
    // vs 0.182 ms, so short columns stay on the 128-bit direct kernel)
    if (BO_ACROSS_TMA && n >= 64 && p % 4 == 0 && aligned16(src) && aligned16(dst) && p >= 2LL * 128 * num_sms() &&
        p < (int64_t(1) << 31) && n < (int64_t(1) << 31))
        return launch_across_tma<T, 128>(src, dst, n, p, st);
    // too few instances for 128-wide blocks but long columns (the paper's n = 32K,
    // p = 8K): 32-wide blocks with a 12-deep ring keep every SM streaming
    // (measured: n = 32K p = 8K 0.383 vs 1.644 ms with the scalar kernel, 5.6 TB/s;
    // n = 1024 p = 16384 29 vs 61 us; n = 4096 p = 8192 52 vs 211 us)
    if (BO_ACROSS_TMA && n >= 256 && p % 4 == 0 && p >= 32 && aligned16(src) && aligned16(dst) &&
        p < (int64_t(1) << 31) && n < (int64_t(1) << 31) && p / 4 < 512LL * num_sms())
        return launch_across_tma<T, 32>(src, dst, n, p, st);
    // 128-bit lanes when there are enough instances to fill the GPU with
    // 4-instance threads; otherwise one instance per thread, 16 rows in flight
    if (p % 4 == 0 && aligned16(src) && aligned16(dst) && p / 4 >= 512LL * num_sms()) {
        const long long p4 = p / 4;
        const unsigned grid = static_cast<unsigned>((p4 + 255) / 256);
#ifndef BO_ACROSS_U
#define BO_ACROSS_U 8
#endif
        launch(ps_across_vec4<T, BO_ACROSS_U>, grid, 256, 0, st, src, dst, n, p4);
        return after_launch("ps_across_vec4");
    }
    const unsigned grid = static_cast<unsigned>((p + 255) / 256);
    launch(ps_across_scalar<T, 16>, grid, 256, 0, st, src, dst, n, p);
    return after_launch("ps_across_scalar");
}

template <typename T, int INST>
static int launch_fused_row_tma(const T *src, T *dst, int64_t n, int64_t p, cudaStream_t st) {
    using C = fr::Cfg<INST>;
    CUtensorMap smap, dmap;
    if (!make_tmap_2d(&smap, src, p, n, INST, fr::kElems, CU_TENSOR_MAP_SWIZZLE_128B) ||
        !make_tmap_2d(&dmap, dst, p, n, INST, fr::kElems, CU_TENSOR_MAP_SWIZZLE_128B))
        return fail(BO_ECUDA, "prefix fused-row: cuTensorMapEncodeTiled failed");
    const bool attr = ensure_dyn_smem(reinterpret_cast<const void *>(&ps_fused_row_tma<T, INST>), static_cast<int>(C::kSmem));
    if (!attr) return fail(BO_ECUDA, "prefix fused-row: cannot set dynamic smem");
    const long long ntiles = (p + INST - 1) / INST;
    const int nchunks = static_cast<int>((n + fr::kElems - 1) / fr::kElems);
    int per_sm = 1;
    per_sm = max_blocks_per_sm(reinterpret_cast<const void *>(&ps_fused_row_tma<T, INST>), INST, C::kSmem);
    const long long grid = std::min<long long>(ntiles, static_cast<long long>(std::max(per_sm, 1)) * num_sms());
    const int slot = work_slot_for(st);
    launch(ps_fused_row_tma<T, INST>, static_cast<unsigned>(grid), INST, C::kSmem, st, smap, dmap, ntiles, nchunks,
                                                                                   slot);
    return after_launch("ps_fused_row_tma");
}

template <typename T>
static int launch_fused_row(const T *src, T *dst, int64_t n, int64_t p, cudaStream_t st) {
    if (fused_tma_ok(src, dst, n, p)) {
        if (p < 2LL * 128 * num_sms()) return launch_fused_row_tma<T, 32>(src, dst, n, p, st);
        return launch_fused_row_tma<T, 128>(src, dst, n, p, st);
    }
    const long long blocks = std::min<long long>((p + 127) / 128, 16LL * num_sms());
    launch(ps_fused_row_smem<T>, static_cast<unsigned>(blocks), 128, 0, st, src, dst, n, p);
    return after_launch("ps_fused_row_smem");
}

template <typename T>
static int launch_warpscan(const T *src, T *dst, int64_t n, int64_t p, cudaStream_t st) {
    const long long blocks = std::min<long long>((p + 7) / 8, 32LL * num_sms());
    if (n % 4 == 0 && aligned16(src) && aligned16(dst))
        launch(ps_warpscan<T, true>, static_cast<unsigned>(blocks), 256, 0, st, src, dst, n, p);
    else
        launch(ps_warpscan<T, false>, static_cast<unsigned>(blocks), 256, 0, st, src, dst, n, p);
    return after_launch("ps_warpscan");
}

template <typename T>
static int run_prefix(const T *src, T *dst, int64_t n, int64_t p, int layout, int variant, void *ws,
                      cudaStream_t st) {
    switch (variant) {
        case BO_PS_ACROSS:
            return launch_across(src, dst, n, p, st);
        case BO_PS_FUSED_ROW:
            return launch_fused_row(src, dst, n, p, st);
        case BO_PS_WARPSCAN:
            return launch_warpscan(src, dst, n, p, st);
        case BO_PS_TRANSPOSED: {
            // row-wise [p][n] -> column-wise [n][p] in ws -> ACROSS in place -> back into dst
            int rc = launch_transpose(src, ws, p, n, st);
            if (rc) return rc;
            rc = launch_across(static_cast<const T *>(ws), static_cast<T *>(ws), n, p, st);
            if (rc) return rc;
            return launch_transpose(ws, dst, n, p, st);
        }
        case BO_PS_NAIVE: {
            const unsigned grid = static_cast<unsigned>((p + 63) / 64);
            launch(ps_naive<T>, grid, 64, 0, st, src, dst, n, p, layout);
            return after_launch("ps_naive");
        }
        default:
            return fail(BO_EINVAL, "prefix: unknown variant");
    }
}

int prefix_dispatch(const void *src, void *dst, int64_t n, int64_t p, int dtype, int layout, int variant,
                    void *ws, cudaStream_t st) {
    if (dtype == BO_I32)
        return run_prefix(static_cast<const int32_t *>(src), static_cast<int32_t *>(dst), n, p, layout,
                          variant, ws, st);
    return run_prefix(static_cast<const float *>(src), static_cast<float *>(dst), n, p, layout, variant, ws,
                      st);
}

}  // namespace bo
