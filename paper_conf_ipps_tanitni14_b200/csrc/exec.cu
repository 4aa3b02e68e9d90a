// exec.cu -- generic bulk executor of oblivious programs (NEXT-3; Theorem 2,
// P:132-137): p threads each run the same straight-line program on their own
// instance memory, in the row-wise (j*msize + a) or column-wise (a*p + j)
// arrangement.  The instruction stream is read once per warp
// (uniform broadcast loads through L1), registers live in shared memory
// ([r][thread], conflict-free), and every LOAD/STORE of a warp touches one
// address group column-wise or 32 groups row-wise -- exactly the Theorem 2
// comparison.  Encoding: see include/bulkobl.h / programs.py.
//
// A plain interpreter is bound by its per-instruction dispatch (uniform fetch,
// branch tree, shared-memory register file: 70-90 SASS instructions per
// program instruction, measured), so
// (1) the host rewrites straight-line patterns into single internal
//     instructions before upload (exec_device_program; every memory word ends
//     with the value the original sequence gives -- registers are not
//     observable afterwards, so dead ones are not written back);
// (2) runs of the two hot forms (CE2, ACC_ADD below) execute in tight loops of
//     their own, in groups whose memory operands are all loaded first (several
//     loads in flight per warp; a load of an address an earlier member of the
//     group stores to takes the stored value), fetching the next word ahead;
// (3) when the CTA's 128 instance memories fit (exec_staged_smem) they are
//     staged in shared memory with coalesced copies, so every LOAD/STORE is a
//     conflict-free shared access in either arrangement; when they do not, a
//     program with address locality is cut into windows (WIN words, see
//     exec_device_program) and each window is staged the same way (row-wise
//     only: column-wise accesses are already coalesced and measured faster).
// The internal instructions:
//   CE  = LOAD ra,A; LOAD rb,B; MIN rn,..; MAX rx,..; STORE S1,q1; STORE S2,q2
//         (a compare-exchange: the whole bitonic network, programs.py), two
//         words: (8, A, B, regs | order bits), (S1, S2, q1 | q2 << 2, 0);
//   LOS = LOAD rl,A; OP rd,ry,rz; STORE S,rs   (OP = ADD/SUB/MIN/MAX; the
//         prefix program is one per element), one word (9 + OP - ADD, A, S,
//         rl | rd << 6 | ry << 12 | rz << 18 | rs << 24 | live bits 30, 31).
// Both write back only the registers still live afterwards.  Two lean forms
// take the common cases with one word and no register traffic:
//   CE2 = an in-place compare-exchange (the two STOREs put MIN and MAX back on
//         the two loaded addresses, no register live afterwards -- every
//         comparator of the bitonic network): (13, X, Y, order bits), b[X] <-
//         the MIN, b[Y] <- the MAX, bit 0 / bit 1: the MIN's / MAX's first
//         operand is b[Y] (else b[X]);
//   ACC_ADD = LOAD t,A; ADD r,r,t (either order); STORE S,r with t dead
//         afterwards (the prefix program's step): (14, A, S, r).
//         a + b is exactly b + a in IEEE-754 and in wrapping int32, and the
//         GPU's NaN result carries no operand payload.
#include "common.cuh"

#include <algorithm>
#include <climits>
#include <vector>

#include "exec.h"

namespace bo {

// fetch the next word of a run before executing the current one (A/B switch)
#ifndef BO_EX_RUN_FETCH
#define BO_EX_RUN_FETCH 1
#endif

// ACC_ADD steps whose memory operands are loaded together (A/B switch; 1 = off)
#ifndef BO_EX_ACC_GROUP
#define BO_EX_ACC_GROUP 8
#endif
#ifndef BO_EX_WINDOW_COL
#define BO_EX_WINDOW_COL 0
#endif
#ifndef BO_EX_CE_GROUP
#define BO_EX_CE_GROUP 2
#endif

namespace ex {
enum { LOAD = 0, STORE, ADD, SUB, MIN, MAX, MOV, CONST, CE, LOS_ADD, LOS_SUB, LOS_MIN, LOS_MAX, CE2, ACC_ADD, WIN };
constexpr int kThreads = 128;
constexpr int kPitch = kThreads + 1;
}

// Shared memory of the staged kernel (0: run direct).  The cap keeps >= 3 CTAs
// (12 warps) per SM.
size_t exec_staged_smem(int64_t msize, int nregs) {
    const size_t b = (static_cast<size_t>(nregs) * ex::kThreads + static_cast<size_t>(msize) * ex::kPitch) * 4;
    return msize > 0 && b <= 72 * 1024 ? b : 0;
}

// Windowed staging: words of a window, so registers + window fit 64 KB (>= 3 CTAs per SM)
static int exec_window_cap(int nregs) {
    const int w = (64 * 1024 / 4 - nregs * ex::kThreads) / ex::kPitch;
    return w < 64 ? w : 64;
}

// ---- host: the uploaded program (patterns above fused; the rest verbatim)
// Registers are not observable after the program (only memory is), so a fused
// instruction writes back only the registers a later instruction reads before
// overwriting them: live_after[i] = registers live after original instruction i.
static std::vector<int32_t> exec_fuse(const int32_t *prog, int64_t t) {
    auto op = [&](int64_t i) { return i < t ? prog[4 * i] : -1; };
    auto f = [&](int64_t i, int k) { return prog[4 * i + k]; };
    std::vector<uint64_t> live_after(static_cast<size_t>(t));
    uint64_t live = 0;
    for (int64_t i = t - 1; i >= 0; --i) {
        live_after[i] = live;
        const int o = op(i), x = f(i, 1), y = f(i, 2), z = f(i, 3);
        uint64_t rd = 0, wr = 0;
        switch (o) {
            case ex::LOAD: wr = 1ull << x; break;
            case ex::STORE: rd = 1ull << y; break;
            case ex::MOV: wr = 1ull << x; rd = 1ull << y; break;
            case ex::CONST: wr = 1ull << x; break;
            default: wr = 1ull << x; rd = (1ull << y) | (1ull << z); break;   // ADD SUB MIN MAX
        }
        live = (live & ~wr) | rd;
    }
    auto is_live = [&](int64_t i, int r) { return static_cast<int>((live_after[i] >> r) & 1); };
    std::vector<int32_t> out;
    out.reserve(static_cast<size_t>(4 * t));
    int64_t i = 0;
    while (i < t) {
        // CE: two LOADs into distinct registers, MIN and MAX over exactly those two
        // (either operand order) into two further distinct registers, two STOREs of
        // any of the four
        if (i + 5 < t && op(i) == ex::LOAD && op(i + 1) == ex::LOAD && op(i + 2) == ex::MIN && op(i + 3) == ex::MAX &&
            op(i + 4) == ex::STORE && op(i + 5) == ex::STORE) {
            const int ra = f(i, 1), rb = f(i + 1, 1), rn = f(i + 2, 1), rx = f(i + 3, 1);
            const int y1 = f(i + 2, 2), z1 = f(i + 2, 3), y2 = f(i + 3, 2), z2 = f(i + 3, 3);
            const bool regs_ok = ra != rb && rn != ra && rn != rb && rx != ra && rx != rb && rx != rn;
            const bool min_ok = (y1 == ra && z1 == rb) || (y1 == rb && z1 == ra);
            const bool max_ok = (y2 == ra && z2 == rb) || (y2 == rb && z2 == ra);
            auto sel = [&](int r) { return r == ra ? 0 : r == rb ? 1 : r == rn ? 2 : r == rx ? 3 : -1; };
            const int q1 = sel(f(i + 4, 2)), q2 = sel(f(i + 5, 2));
            const int A = f(i, 2), B = f(i + 1, 2), S1 = f(i + 4, 1), S2 = f(i + 5, 1);
            const bool dead = !is_live(i + 5, ra) && !is_live(i + 5, rb) && !is_live(i + 5, rn) && !is_live(i + 5, rx);
            if (regs_ok && min_ok && max_ok && dead && A != B && S1 != S2 && ((q1 == 2 && q2 == 3) || (q1 == 3 && q2 == 2)) &&
                ((S1 == A && S2 == B) || (S1 == B && S2 == A))) {
                const int X = q1 == 2 ? S1 : S2, Y = q1 == 2 ? S2 : S1;        // b[X] <- MIN, b[Y] <- MAX
                const int ry = X == A ? rb : ra;                                 // the register b[Y] was loaded into
                out.insert(out.end(), {ex::CE2, X, Y, (y1 == ry ? 1 : 0) | (y2 == ry ? 2 : 0)});
                i += 6;
                continue;
            }
            if (regs_ok && min_ok && max_ok && q1 >= 0 && q2 >= 0) {
                const int bits = ra | (rb << 6) | (rn << 12) | (rx << 18) | ((y1 == rb) << 24) | ((y2 == rb) << 25) |
                                 (is_live(i + 5, ra) << 26) | (is_live(i + 5, rb) << 27) |
                                 (is_live(i + 5, rn) << 28) | (is_live(i + 5, rx) << 29);
                out.insert(out.end(), {ex::CE, f(i, 2), f(i + 1, 2), bits, f(i + 4, 1), f(i + 5, 1), q1 | (q2 << 2), 0});
                i += 6;
                continue;
            }
        }
        // LOS: LOAD, a two-operand op, STORE
        if (i + 2 < t && op(i) == ex::LOAD && op(i + 1) >= ex::ADD && op(i + 1) <= ex::MAX && op(i + 2) == ex::STORE) {
            const int rl = f(i, 1), rd = f(i + 1, 1), ry = f(i + 1, 2), rz = f(i + 1, 3), rs = f(i + 2, 2);
            const int wl = rl != rd && is_live(i + 2, rl), wd = is_live(i + 2, rd);
            if (op(i + 1) == ex::ADD && rl != rd && rs == rd && !wl &&
                ((ry == rd && rz == rl) || (ry == rl && rz == rd))) {
                out.insert(out.end(), {ex::ACC_ADD, f(i, 2), f(i + 2, 1), rd});
                i += 3;
                continue;
            }
            out.insert(out.end(), {ex::LOS_ADD + (op(i + 1) - ex::ADD), f(i, 2), f(i + 2, 1),
                                   static_cast<int32_t>(static_cast<uint32_t>(rl | (rd << 6) | (ry << 12) | (rz << 18) |
                                                                              (rs << 24)) |
                                                        (static_cast<uint32_t>(wl) << 30) |
                                                        (static_cast<uint32_t>(wd) << 31))});
            i += 3;
            continue;
        }
        out.insert(out.end(), {f(i, 0), f(i, 1), f(i, 2), f(i, 3)});
        ++i;
    }
    return out;
}

// Windows (instance memories too large to stage whole, exec_staged_smem == 0):
// the fused program is cut greedily into segments whose addresses span at most
// exec_window_cap words, each preceded by WIN (15, lo, len, 0); the kernel then
// keeps [lo, lo+len) of its 128 instances in shared memory, copying it in (and
// the previous window out, if stored to) with coalesced row segments.  Used
// only when every instruction fits a window and the copies move at most twice
// the words the program's own LOADs and STOREs touch (so a program that jumps
// around its memory keeps the direct path).
ExecProgram exec_device_program(const int32_t *prog, int64_t t, int64_t msize, int nregs) {
    ExecProgram ep;
    ep.words = exec_fuse(prog, t);
    ep.wmax = 0;
    if (msize <= 0 || exec_staged_smem(msize, nregs) != 0) return ep;
    const int cap = exec_window_cap(nregs);
    if (cap < 8) return ep;
    const std::vector<int32_t> &w = ep.words;
    const size_t nw = w.size() / 4;
    // addresses of fused word i (second word of CE handled with its first)
    struct Seg { size_t begin, end; int lo, hi; };
    std::vector<Seg> segs;
    long long direct = 0, copies = 0;
    Seg cur{0, 0, INT32_MAX, -1};
    bool stores = false;
    auto close = [&](size_t end) {
        cur.end = end;
        if (cur.hi >= cur.lo) copies += static_cast<long long>(cur.hi - cur.lo + 1) * (stores ? 2 : 1);
        segs.push_back(cur);
        stores = false;
    };
    for (size_t i = 0; i < nw;) {
        const int o = w[4 * i];
        int a[4], na = 0, nst = 0;
        size_t len = 1;
        switch (o) {
            case ex::LOAD: a[na++] = w[4 * i + 2]; break;
            case ex::STORE: a[na++] = w[4 * i + 1]; nst = 1; break;
            case ex::CE: a[na++] = w[4 * i + 1]; a[na++] = w[4 * i + 2]; a[na++] = w[4 * i + 4];
                         a[na++] = w[4 * i + 5]; nst = 2; len = 2; break;
            case ex::LOS_ADD: case ex::LOS_SUB: case ex::LOS_MIN: case ex::LOS_MAX:
            case ex::ACC_ADD: a[na++] = w[4 * i + 1]; a[na++] = w[4 * i + 2]; nst = 1; break;
            case ex::CE2: a[na++] = w[4 * i + 1]; a[na++] = w[4 * i + 2]; nst = 2; break;
            default: break;
        }
        int lo = cur.lo, hi = cur.hi, ilo = INT32_MAX, ihi = -1;
        for (int k = 0; k < na; ++k) {
            ilo = std::min(ilo, a[k]);
            ihi = std::max(ihi, a[k]);
        }
        if (na > 0 && ihi - ilo + 1 > cap) { ep.wmax = 0; return ep; }   // one instruction spans too much
        if (na > 0) {
            lo = std::min(lo, ilo);
            hi = std::max(hi, ihi);
            if (hi - lo + 1 > cap) {                                     // start a new window here
                close(i);
                cur = Seg{i, 0, ilo, ihi};
            } else {
                cur.lo = lo;
                cur.hi = hi;
            }
            direct += na;
            stores = stores || nst > 0;
        }
        i += len;
    }
    close(nw);
    // worth it only with enough work per window, and never longer than the
    // caller's program (the device buffer holds 16*t bytes)
    if (copies > 2 * direct || static_cast<long long>(segs.size()) * 8 > direct ||
        ep.words.size() + 4 * segs.size() > static_cast<size_t>(4 * t))
        return ep;
    std::vector<int32_t> out;
    out.reserve(w.size() + 4 * segs.size());
    for (const Seg &sg : segs) {
        if (sg.hi >= sg.lo) {
            out.insert(out.end(), {ex::WIN, sg.lo, sg.hi - sg.lo + 1, 0});
            ep.wmax = std::max(ep.wmax, sg.hi - sg.lo + 1);
        }
        out.insert(out.end(), w.begin() + 4 * sg.begin, w.begin() + 4 * sg.end);
    }
    ep.words.swap(out);
    return ep;
}

template <typename T>
__device__ __forceinline__ T ex_add(T a, T b) { return add_wrap(a, b); }
__device__ __forceinline__ int32_t ex_sub(int32_t a, int32_t b) {
    return static_cast<int32_t>(static_cast<uint32_t>(a) - static_cast<uint32_t>(b));
}
__device__ __forceinline__ float ex_sub(float a, float b) { return __fsub_rn(a, b); }

// Instance memory.  Direct: LOAD/STORE go to global memory in the caller's
// arrangement.  STAGED (msize small enough, exec_staged_smem): the CTA copies
// its 128 instances' memories into shared memory as [a][thread] (pitch
// kThreads + 1, so the row-wise transposing copy is conflict-free too) with
// coalesced loads, interprets against it, and copies every word back -- the
// row-wise arrangement then costs what the column-wise one does (P:122-126's
// difference is paid once, coalesced, instead of on every access).
// WINDOWED: the same for the window [wlo, wlo + wlen) the last WIN named.
enum { EX_DIRECT = 0, EX_STAGED = 1, EX_WINDOWED = 2 };

template <typename T, int LAYOUT, int MODE>
__global__ void __launch_bounds__(ex::kThreads)
exec_kernel(const int4 *__restrict__ prog, long long t, T *mem, long long msize, long long p, int nregs, int nzero) {
    pdl_begin();
    constexpr bool STAGED = MODE == EX_STAGED;
    extern __shared__ uint8_t smem_raw[];
    T *R = reinterpret_cast<T *>(smem_raw) + threadIdx.x;     // r[x] at R[x * kThreads]
    T *Mb = reinterpret_cast<T *>(smem_raw) + nregs * ex::kThreads;
    constexpr int kPitch = ex::kPitch;
    T *M = Mb + threadIdx.x;                                    // staged b[a] at M[a * kPitch]
    int wlo = 0, wlen = 0;                                      // WINDOWED: current window
    bool dirty = false;
    const long long j0 = blockIdx.x * static_cast<long long>(ex::kThreads);
    const long long j = j0 + threadIdx.x;
    const bool live = j < p;
    const int cnt = static_cast<int>(p - j0 < ex::kThreads ? p - j0 : ex::kThreads);
    const int ms = static_cast<int>(msize);
    auto addr = [&](long long a) -> long long { return LAYOUT == BO_ROW_WISE ? j * msize + a : a * p + j; };
    auto ld = [&](int a) -> T {
        if constexpr (STAGED) return M[a * kPitch];
        else if constexpr (MODE == EX_WINDOWED) return M[(a - wlo) * kPitch];
        else return live ? mem[addr(a)] : T(0);
    };
    auto st = [&](int a, T v) {
        if constexpr (STAGED) M[a * kPitch] = v;
        else if constexpr (MODE == EX_WINDOWED) { M[(a - wlo) * kPitch] = v; dirty = true; }
        else if (live) mem[addr(a)] = v;
    };
    // WINDOWED: copy the window out / in, coalesced (row-wise: one warp per
    // instance row segment; column-wise: one warp per address row)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    auto window_out = [&]() {
        if (LAYOUT == BO_ROW_WISE) {
            for (int jl = warp; jl < cnt; jl += ex::kThreads / 32) {
                T *g = mem + (j0 + jl) * msize + wlo;
                for (int a = lane; a < wlen; a += 32) g[a] = Mb[a * kPitch + jl];
            }
        } else {
            for (int a = 0; a < wlen; ++a)
                if (live) mem[(wlo + a) * p + j] = M[a * kPitch];
        }
    };
    auto window_in = [&]() {
        if (LAYOUT == BO_ROW_WISE) {
            // all of a thread's loads first (up to 2 x 32 in flight), then the stores
            constexpr int kRows = ex::kThreads / (ex::kThreads / 32);   // 32 instance rows per warp
            for (int a0 = 0; a0 < wlen; a0 += 32) {
                const int a = a0 + lane;
                T v[kRows];
#pragma unroll
                for (int r = 0; r < kRows; ++r) {
                    const int jl = warp + r * (ex::kThreads / 32);
                    v[r] = jl < cnt && a < wlen ? mem[(j0 + jl) * msize + wlo + a] : T(0);
                }
#pragma unroll
                for (int r = 0; r < kRows; ++r)
                    if (a < wlen) Mb[a * kPitch + warp + r * (ex::kThreads / 32)] = v[r];
            }
        } else {
#pragma unroll 8
            for (int a = 0; a < wlen; ++a) M[a * kPitch] = live ? mem[(wlo + a) * p + j] : T(0);
        }
    };
    if constexpr (STAGED) {
        if (LAYOUT == BO_ROW_WISE) {                            // cnt*msize contiguous words
            const T *g = mem + j0 * msize;
            const int total = cnt * ms;
            for (int e = threadIdx.x; e < total; e += ex::kThreads) {
                const int jl = e / ms, a = e - jl * ms;
                Mb[a * kPitch + jl] = g[e];
            }
        } else {
            for (int a = 0; a < ms; ++a)
                if (live) M[a * kPitch] = mem[a * p + j];
        }
        if (!live)
            for (int a = 0; a < ms; ++a) M[a * kPitch] = T(0);
        __syncthreads();
    }
    // registers start at 0 (bulkobl.h); the host passes nzero = 0 when the program
    // writes every register before reading it (every builder in programs.py does)
    for (int x = 0; x < nzero; ++x) R[x * ex::kThreads] = T(0);
    for (long long i = 0; i < t;) {
        int4 ins = __ldg(prog + i);                            // same address for the whole warp
        // runs of the two hot forms execute in their own tight loops: no dispatch
        // between consecutive words of one form
        if (ins.x == ex::CE2) {
            // groups of BO_EX_CE_GROUP comparators: all operands loaded first, a load
            // of an address an earlier comparator of the group stores to forwarded
            while (BO_EX_CE_GROUP > 1 && i + BO_EX_CE_GROUP <= t) {
                constexpr int G = BO_EX_CE_GROUP > 1 ? BO_EX_CE_GROUP : 2;
                int4 w[G];
                w[0] = ins;
                bool all = true;
#pragma unroll
                for (int k = 1; k < G; ++k) {
                    w[k] = __ldg(prog + i + k);
                    all = all && w[k].x == ex::CE2;
                }
                if (!all) break;
                T vx[G], vy[G], mn[G], mx[G];
#pragma unroll
                for (int k = 0; k < G; ++k) {
                    vx[k] = ld(w[k].y);
                    vy[k] = ld(w[k].z);
                }
#pragma unroll
                for (int k = 0; k < G; ++k) {
                    T a = vx[k], b = vy[k];
#pragma unroll
                    for (int q = 0; q < k; ++q) {                // latest earlier store wins
                        if (w[q].y == w[k].y) a = mn[q];
                        if (w[q].z == w[k].y) a = mx[q];
                        if (w[q].y == w[k].z) b = mn[q];
                        if (w[q].z == w[k].z) b = mx[q];
                    }
                    const int z = w[k].w;
                    const T my = z & 1 ? b : a, mz = z & 1 ? a : b;
                    const T xy = z & 2 ? b : a, xz = z & 2 ? a : b;
                    mn[k] = mz < my ? mz : my;
                    mx[k] = xy < xz ? xz : xy;
                    st(w[k].y, mn[k]);
                    st(w[k].z, mx[k]);
                }
                i += G;
                if (i < t) ins = __ldg(prog + i);
                if (i >= t || ins.x != ex::CE2) break;
            }
            if (i >= t || ins.x != ex::CE2) continue;
            do {
                const int x = ins.y, y = ins.z, z = ins.w;
                const T vx = ld(x), vy = ld(y);
                const T my = z & 1 ? vy : vx, mz = z & 1 ? vx : vy;
                const T xy = z & 2 ? vy : vx, xz = z & 2 ? vx : vy;
                const int4 nx = BO_EX_RUN_FETCH && i + 1 < t ? __ldg(prog + i + 1) : ins;
                st(x, mz < my ? mz : my);
                st(y, xy < xz ? xz : xy);
                if (++i < t) ins = BO_EX_RUN_FETCH ? nx : __ldg(prog + i);
            } while (i < t && ins.x == ex::CE2);
            continue;
        }
        if (ins.x == ex::ACC_ADD) {
            // groups of kAccGroup: all their memory operands are loaded first (that
            // many loads in flight instead of one); a load whose address an earlier
            // step of the group stores to takes that stored value instead
            while (BO_EX_ACC_GROUP > 1 && i + BO_EX_ACC_GROUP <= t) {
                constexpr int G = BO_EX_ACC_GROUP > 1 ? BO_EX_ACC_GROUP : 2;
                int4 w[G];
                w[0] = ins;
                bool all = true, one_acc = true;
#pragma unroll
                for (int k = 1; k < G; ++k) {
                    w[k] = __ldg(prog + i + k);
                    all = all && w[k].x == ex::ACC_ADD;
                    one_acc = one_acc && w[k].w == w[0].w;
                }
                if (!all) break;
                T v[G], sv[G];
#pragma unroll
                for (int k = 0; k < G; ++k) v[k] = ld(w[k].y);
                if (one_acc) {                                  // one accumulator: kept in a register
                    T acc = R[w[0].w * ex::kThreads];
#pragma unroll
                    for (int k = 0; k < G; ++k) {
                        T a = v[k];
#pragma unroll
                        for (int q = 0; q < k; ++q)
                            if (w[q].z == w[k].y) a = sv[q];
                        acc = ex_add(acc, a);
                        sv[k] = acc;
                        st(w[k].z, acc);
                    }
                    R[w[0].w * ex::kThreads] = acc;
                } else {
#pragma unroll
                    for (int k = 0; k < G; ++k) {
                        T a = v[k];
#pragma unroll
                        for (int q = 0; q < k; ++q)
                            if (w[q].z == w[k].y) a = sv[q];
                        sv[k] = ex_add(R[w[k].w * ex::kThreads], a);
                        R[w[k].w * ex::kThreads] = sv[k];
                        st(w[k].z, sv[k]);
                    }
                }
                i += G;
                if (i < t) ins = __ldg(prog + i);
                if (i >= t || ins.x != ex::ACC_ADD) break;
            }
            if (i >= t || ins.x != ex::ACC_ADD) continue;
            do {
                const int4 nx = BO_EX_RUN_FETCH && i + 1 < t ? __ldg(prog + i + 1) : ins;
                const T r = ex_add(R[ins.w * ex::kThreads], ld(ins.y));
                R[ins.w * ex::kThreads] = r;
                st(ins.z, r);
                if (++i < t) ins = BO_EX_RUN_FETCH ? nx : __ldg(prog + i);
            } while (i < t && ins.x == ex::ACC_ADD);
            continue;
        }
        const int x = ins.y, y = ins.z, z = ins.w;
        switch (ins.x) {
            case ex::LOAD: R[x * ex::kThreads] = ld(y); break;
            case ex::STORE: st(x, R[y * ex::kThreads]); break;
            case ex::ADD: R[x * ex::kThreads] = ex_add(R[y * ex::kThreads], R[z * ex::kThreads]); break;
            case ex::SUB: R[x * ex::kThreads] = ex_sub(R[y * ex::kThreads], R[z * ex::kThreads]); break;
            case ex::MIN: {                                     // "if r < s then s <- r"
                const T a = R[y * ex::kThreads], b = R[z * ex::kThreads];
                R[x * ex::kThreads] = b < a ? b : a;
                break;
            }
            case ex::MAX: {
                const T a = R[y * ex::kThreads], b = R[z * ex::kThreads];
                R[x * ex::kThreads] = a < b ? b : a;
                break;
            }
            case ex::MOV: R[x * ex::kThreads] = R[y * ex::kThreads]; break;
            case ex::WIN:                                       // (15, lo, len): switch windows
                if constexpr (MODE == EX_WINDOWED) {
                    __syncthreads();
                    if (dirty) window_out();
                    wlo = x;
                    wlen = y;
                    dirty = false;
                    window_in();
                    __syncthreads();
                }
                break;
            case ex::CONST: {
                const uint32_t u = static_cast<uint32_t>(y);
                R[x * ex::kThreads] = *reinterpret_cast<const T *>(&u);
                break;
            }
            case ex::CE: {                                      // two words (see the header)
                const int4 w2 = __ldg(prog + i + 1);
                ++i;
                const T va = ld(x), vb = ld(y);
                // MIN r <- (r[z'] < r[y'] ? r[z'] : r[y']); MAX r <- (r[y'] < r[z'] ? r[z'] : r[y'])
                const T my = (z >> 24) & 1 ? vb : va, mz = (z >> 24) & 1 ? va : vb;
                const T xy = (z >> 25) & 1 ? vb : va, xz = (z >> 25) & 1 ? va : vb;
                const T mn = mz < my ? mz : my, mx = xy < xz ? xz : xy;
                if ((z >> 26) & 1) R[(z & 63) * ex::kThreads] = va;             // live-out registers only
                if ((z >> 27) & 1) R[((z >> 6) & 63) * ex::kThreads] = vb;
                if ((z >> 28) & 1) R[((z >> 12) & 63) * ex::kThreads] = mn;
                if ((z >> 29) & 1) R[((z >> 18) & 63) * ex::kThreads] = mx;
                const int q1 = w2.z & 3, q2 = (w2.z >> 2) & 3;
                st(w2.x, q1 == 0 ? va : q1 == 1 ? vb : q1 == 2 ? mn : mx);
                st(w2.y, q2 == 0 ? va : q2 == 1 ? vb : q2 == 2 ? mn : mx);
                break;
            }
            case ex::LOS_ADD:
            case ex::LOS_SUB:
            case ex::LOS_MIN:
            case ex::LOS_MAX: {                                 // LOAD rl,x; OP rd,ry,rz; STORE y,rs
                const int rl = z & 63, rd = (z >> 6) & 63, ry = (z >> 12) & 63, rz = (z >> 18) & 63, rs = (z >> 24) & 63;
                const T v = ld(x);
                const T a = ry == rl ? v : R[ry * ex::kThreads], b = rz == rl ? v : R[rz * ex::kThreads];
                T r;
                switch (ins.x) {
                    case ex::LOS_ADD: r = ex_add(a, b); break;
                    case ex::LOS_SUB: r = ex_sub(a, b); break;
                    case ex::LOS_MIN: r = b < a ? b : a; break;
                    default: r = a < b ? b : a; break;
                }
                // the stored value is read before the live-out write-backs (rs may be
                // neither rd nor rl: then it is an older register, unchanged here)
                const T sv = rs == rd ? r : rs == rl ? v : R[rs * ex::kThreads];
                if ((z >> 30) & 1) R[rl * ex::kThreads] = v;
                if ((z >> 31) & 1) R[rd * ex::kThreads] = r;
                st(y, sv);
                break;
            }
            default: break;
        }
        ++i;
    }
    if constexpr (MODE == EX_WINDOWED) {
        __syncthreads();
        if (dirty) window_out();
    }
    if constexpr (STAGED) {
        __syncthreads();
        if (LAYOUT == BO_ROW_WISE) {
            T *g = mem + j0 * msize;
            const int total = cnt * ms;
            for (int e = threadIdx.x; e < total; e += ex::kThreads) {
                const int jl = e / ms, a = e - jl * ms;
                g[e] = Mb[a * kPitch + jl];
            }
        } else {
            for (int a = 0; a < ms; ++a)
                if (live) mem[a * p + j] = M[a * kPitch];
        }
    }
}

template <typename T, int LAYOUT>
static void launch_exec_t(const int4 *pg, int64_t t, T *mem, int64_t msize, int64_t p, int nregs, int nzero,
                          int wmax, unsigned grid, cudaStream_t st) {
    const size_t staged = exec_staged_smem(msize, nregs);
    const size_t windowed = (static_cast<size_t>(nregs) * ex::kThreads + static_cast<size_t>(wmax) * ex::kPitch) * 4;
    if (staged && ensure_dyn_smem(reinterpret_cast<const void *>(exec_kernel<T, LAYOUT, EX_STAGED>), static_cast<int>(staged)))
        launch(exec_kernel<T, LAYOUT, EX_STAGED>, grid, ex::kThreads, staged, st, pg, (long long)t, mem,
               (long long)msize, (long long)p, nregs, nzero);
    else if (wmax > 0 && (BO_EX_WINDOW_COL || LAYOUT == BO_ROW_WISE) && ensure_dyn_smem(reinterpret_cast<const void *>(exec_kernel<T, LAYOUT, EX_WINDOWED>),
                                         static_cast<int>(windowed)))
        launch(exec_kernel<T, LAYOUT, EX_WINDOWED>, grid, ex::kThreads, windowed, st, pg, (long long)t, mem,
               (long long)msize, (long long)p, nregs, nzero);
    else
        launch(exec_kernel<T, LAYOUT, EX_DIRECT>, grid, ex::kThreads, static_cast<size_t>(nregs) * ex::kThreads * 4, st,
               pg, (long long)t, mem, (long long)msize, (long long)p, nregs, nzero);
}

int launch_exec(const void *prog, int64_t t, void *mem, int64_t msize, int64_t p, int dtype, int layout, int nregs,
                int nzero, int wmax, cudaStream_t st) {
    const unsigned grid = static_cast<unsigned>((p + ex::kThreads - 1) / ex::kThreads);
    const int4 *pg = static_cast<const int4 *>(prog);
    if (dtype == BO_F32) {
        if (layout == BO_ROW_WISE) launch_exec_t<float, BO_ROW_WISE>(pg, t, static_cast<float *>(mem), msize, p, nregs, nzero, wmax, grid, st);
        else launch_exec_t<float, BO_COLUMN_WISE>(pg, t, static_cast<float *>(mem), msize, p, nregs, nzero, wmax, grid, st);
    } else {
        if (layout == BO_ROW_WISE) launch_exec_t<int32_t, BO_ROW_WISE>(pg, t, static_cast<int32_t *>(mem), msize, p, nregs, nzero, wmax, grid, st);
        else launch_exec_t<int32_t, BO_COLUMN_WISE>(pg, t, static_cast<int32_t *>(mem), msize, p, nregs, nzero, wmax, grid, st);
    }
    return after_launch("exec_kernel");
}

}  // namespace bo
