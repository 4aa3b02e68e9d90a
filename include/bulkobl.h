/*
 * bulkobl.h -- C ABI of libbulkobl.so: bulk execution of oblivious sequential
 * algorithms on NVIDIA B200 (sm_100a).
 *
 * Paper: K. Tani, D. Takafuji, K. Nakano, Y. Ito, "Bulk Execution of Oblivious
 * Algorithms on the Unified Memory Machine, with GPU Implementation",
 * IPDPS Workshops 2014.  "P:<line>" = line of the paper text.
 *
 * The library runs ONE sequential oblivious algorithm on p independent inputs
 * ("bulk execution").  Two algorithms are provided -- inclusive
 * prefix sums (Algorithm Prefix-sums) and the minimum-weight convex
 * polygon triangulation (Algorithm OPT) -- plus the row-wise <->
 * column-wise layout transpose.
 *
 * Conventions for every entry point
 *   - All data pointers are DEVICE pointers (cudaMalloc / torch CUDA tensors)
 *     unless the name ends in _host.  The caller owns every buffer; the
 *     library never allocates, frees or synchronises device memory on the
 *     device entry points.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Device entry points only enqueue work on it (asynchronous);
 *     kernel faults surface at the caller's next synchronisation.
 *   - Return value: BO_OK (0) or a negative bo_status; bulk_last_error()
 *     returns a thread-local message for the last non-OK status.  No C++
 *     exception crosses this boundary.  There is no CPU fallback: every
 *     computation runs in this library's CUDA kernels.
 *   - Element types are 4-byte: BO_I32 (two's-complement int32, addition
 *     wraps mod 2^32) or BO_F32 (IEEE binary32, round to nearest).
 */
#ifndef BULKOBL_H
#define BULKOBL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    BO_OK = 0,
    BO_EINVAL = -1,        /* bad argument: NULL pointer, size out of range,
                              overflow of n*p, partial overlap, short workspace */
    BO_EUNSUPPORTED = -2,  /* a forced variant cannot handle (n, dtype, layout,
                              alignment); BO_AUTO never returns this          */
    BO_ECUDA = -3          /* a CUDA launch / copy failed (message has the
                              cudaGetErrorString text)                         */
} bo_status;

typedef enum {
    BO_ROW_WISE = 0,     /* p rows x n columns: b_j[i] at address j*n + i   */
    BO_COLUMN_WISE = 1,  /* n rows x p columns: b_j[i] at address i*p + j   */
    /* triangulation weights only (NEXT-4): just the K = (n-1)(n-2)/2 weights   */
    /* c[a][b], b - a >= 2, that Algorithm OPT reads, row by row:        */
    /* k(a,b) = a(n-2) - a(a-1)/2 + (b-a-2).                                     */
    BO_PACKED_ROW = 2,   /* c[h*K + k]                                             */
    BO_PACKED_COLUMN = 3 /* c[k*p + h]                                             */
} bo_layout;

typedef enum { BO_I32 = 0, BO_F32 = 1 } bo_dtype;

typedef enum {
    BO_AUTO = 0,
    /* prefix sums */
    BO_PS_ACROSS = 1,      /* column-wise: thread per 4 adjacent instances, 128-bit
                              coalesced rows, sequential in i (bit-exact)          */
    BO_PS_WARPSCAN = 2,    /* row-wise: warp per instance, 128-bit lanes + shuffle
                              scan (fp32 reassociated: not bit-exact)              */
    BO_PS_FUSED_ROW = 3,   /* row-wise: TMA tiles [128 instances x 32 elements]
                              through swizzled smem, one thread per instance scans
                              sequentially (bit-exact), TMA store                  */
    BO_PS_TRANSPOSED = 4,  /* row-wise: transpose -> BO_PS_ACROSS -> transpose,
                              needs an n*p*4-byte workspace (bit-exact)            */
    BO_PS_NAIVE = 5,       /* the paper's GPU kernel: one thread per instance, one
                              32-bit access per step, any layout      */
    /* triangulation */
    BO_TRI_UMM_GLOBAL = 16, /* the paper's Parallel Algorithm OPT: thread per
                               instance, M in global memory in the same
                               arrangement as c; workspace
                               (n-1)^2*p*4 bytes                                  */
    BO_TRI_SMEM_WARP = 17,  /* warp per instance, M in shared memory, diagonal
                               wavefront, k split across lanes + shuffle min      */
    BO_TRI_THREAD_REG = 18, /* thread per instance, M in registers (3 <= n <= 18) */
    BO_TRI_TILED = 19,      /* warp per instance, M in shared memory, 4x4 register
                               tiles (min-plus blocked product), 3 <= n <= 64     */
    BO_TRI_TILED_HALF = 20, /* as BO_TRI_TILED with 16 lanes per instance (two
                               instances per warp)                                 */
    BO_TRI_TILED_GLOBAL = 21, /* CTA per instance, same blocked algorithm, table in a
                               per-CTA global workspace slot kept L2-resident
                               (AUTO for 64 < n < 512); workspace
                               min(p, #SMs) * 16 * (2T^2 + 3T) bytes, T = ceil(n/4),
                               16-byte aligned                                    */
    BO_TRI_TILED_QUARTER = 22, /* as BO_TRI_TILED with 8 lanes per instance (four
                               instances per warp; a lane takes several tiles of a
                               tile-diagonal in turn)                             */
    BO_TRI_TILED_GLOBAL8 = 23 /* CTA per instance, 8x8 register tiles over 8-wide
                               table rows read by 256-bit loads, table in a per-CTA
                               global workspace slot (AUTO for n >= 512);
                               workspace min(p, #SMs) * 32 * (4T^2 + 4T) bytes,
                               T = ceil(n/8), 32-byte aligned                     */
} bo_variant;

/* ------------------------------------------------------------------------- */
/* Inclusive prefix sums of p arrays of n elements (Algorithm Prefix-sums,    */
/* P:95-102; bulk form P:108-118):  dst_j[i] = src_j[0] + ... + src_j[i].     */
/*   src, dst : device, n*p elements in `layout`; dst == src is the paper's   */
/*              in-place form; any other overlap is BO_EINVAL.                */
/*   n >= 0, p >= 0 (n*p == 0 is a no-op); n*p < 2^40.                        */
/*   fp32 sums are accumulated left to right exactly as P:100 for every       */
/*   variant except BO_PS_WARPSCAN.                                           */
/*   workspace: device, >= bulk_prefix_sums_workspace(...) bytes (0 unless    */
/*   the chosen variant is BO_PS_TRANSPOSED); may be NULL when 0 is needed.   */
/* ------------------------------------------------------------------------- */
int bulk_prefix_sums(const void *src, void *dst, int64_t n, int64_t p, int dtype, int layout,
                     int variant, void *workspace, size_t workspace_bytes, void *stream);
size_t bulk_prefix_sums_workspace(int64_t n, int64_t p, int dtype, int layout, int variant);

/* ------------------------------------------------------------------------- */
/* Optimal convex-polygon triangulation of p n-gons (Algorithm OPT, P:174-200;*/
/* bulk form P:215-237).  out[h] = M_h[1, n-1], where                         */
/*   M[i,i] = 0,  M[i,j] = min_{i<=k<j} (M[i,k] + M[k+1,j]) + c[i-1, j].      */
/* That is the minimum total chord weight over all triangulations */
/* PLUS c[0, n-1] (the root side v0 v_{n-1}, which Algorithm OPT adds; set it */
/* to 0 to get the pure chord total).  Only entries c[a][b] with b-a >= 2 are */
/* read: the polygon sides c[a][a+1], the diagonal and the lower triangle    */
/* may hold anything (NaN, inf, garbage) -- they never reach the result.      */
/*   c   : device, dense n x n weights per instance.  Row-wise:               */
/*         c[h*n*n + a*n + b];  column-wise: c[(a*n + b)*p + h], */
/*         or packed (BO_PACKED_ROW / BO_PACKED_COLUMN, see bo_layout).       */
/*   out : device, p elements of dtype.                                       */
/*   n >= 3 (n < 3 is BO_EINVAL), p >= 0; n <= 4096.                          */
/*   The entries read (b-a >= 2) may be negative.  int32 weights must satisfy */
/*   |c| < 2^31 / (2(n-2)) (no overflow); fp32 weights must be finite with    */
/*   |c| < FLT_MAX / (2(n-2)) (no sum overflows).  Results are then           */
/*   bit-identical to the sequential algorithm: min is exact, every sum keeps */
/*   its association, and no table value is ever -0 (reading G16). */
/*   workspace: device, >= bulk_triangulation_workspace(...) bytes; NULL is   */
/*   fine when that is 0.  Needed by BO_TRI_UMM_GLOBAL, BO_TRI_TILED_GLOBAL   */
/*   (16-byte aligned) and BO_TRI_TILED_GLOBAL8 (32-byte aligned), hence by   */
/*   BO_AUTO for every n > 64.  Misaligned or short: BO_EINVAL.  One         */
/*   workspace must not be shared by launches in flight on different streams.*/
/*   Variant n ranges: THREAD_REG 3..18, TILED / TILED_HALF / TILED_QUARTER  */
/*   3..64, SMEM_WARP while one table fits in 200 KB of shared memory,        */
/*   TILED_GLOBAL / GLOBAL8 / UMM_GLOBAL 3..4096; otherwise BO_EUNSUPPORTED.  */
/* ------------------------------------------------------------------------- */
int bulk_triangulation(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout,
                       int variant, void *workspace, size_t workspace_bytes, void *stream);
size_t bulk_triangulation_workspace(int64_t n, int64_t p, int dtype, int layout, int variant);

/* ------------------------------------------------------------------------- */
/* The optimal triangulation itself (NEXT-1; "a few extra bookkeeping steps", */
/* P:157).  out[h] as bulk_triangulation; chords[h] = the n-3 chords of the   */
/* triangulation Algorithm OPT selects when its strict "<" keeps the */
/* FIRST minimising k.  Order: sub-polygons are split depth first from the    */
/* root side (v0, v_{n-1}), left part first; each split of (a, b) at k emits  */
/* (a, k) then (k, b) if that part has >= 3 vertices.                          */
/*   chords : device int16, [p][n-3][2] vertex pairs (a, b), a < b.           */
/*   3 <= n <= 64 (BO_EUNSUPPORTED above), same c layouts and weight          */
/*   preconditions as bulk_triangulation.                                     */
/* ------------------------------------------------------------------------- */
int bulk_triangulation_chords(const void *c, void *out, int16_t *chords, int64_t n, int64_t p, int dtype,
                              int layout, void *stream);

/* ------------------------------------------------------------------------- */
/* Generic bulk execution of an oblivious program (NEXT-3; Theorem 2,         */
/* P:132-137).  p instances each run the same straight-line program of t      */
/* instructions on their own memory of msize words (mem: row-wise            */
/* [p][msize], addr j*msize + a, or column-wise [msize][p], addr a*p + j).    */
/*   prog     : HOST int32 [t][4] = (op, x, y, z):                            */
/*              0 LOAD r[x] <- b[y]        1 STORE b[x] <- r[y]               */
/*              2 ADD  r[x] <- r[y] + r[z] 3 SUB   r[x] <- r[y] - r[z]        */
/*              4 MIN  r[x] <- (r[z] < r[y] ? r[z] : r[y])                     */
/*              5 MAX  r[x] <- (r[y] < r[z] ? r[z] : r[y])                     */
/*              6 MOV  r[x] <- r[y]        7 CONST r[x] <- bit pattern y       */
/*              Registers start at 0; int32 add/sub wrap mod 2^32, fp32 RN.   */
/*              Validated on the host (registers < nregs <= 64, addresses     */
/*              < msize): BO_EINVAL names the first bad instruction.          */
/*   prog_dev : device buffer (16-byte aligned, >= 16*t bytes) the library    */
/*              copies the program into, on `stream`.                         */
/* ------------------------------------------------------------------------- */
int bulk_execute(const int32_t *prog, int64_t t, void *prog_dev, size_t prog_dev_bytes, void *mem, int64_t msize,
                 int64_t p, int dtype, int layout, int nregs, void *stream);

/* ------------------------------------------------------------------------- */
/* Prepared programs: validate, rewrite (the executor's internal              */
/* superinstructions) and upload an oblivious program ONCE, then run it on    */
/* any number of bulk memories with no per-call host work -- and inside CUDA  */
/* graph capture, where bulk_execute can only upload the program unfused.     */
/*   bulk_program_prepare: prog/t/msize/nregs as bulk_execute (same           */
/*     validation, same BO_EINVAL messages); prog_dev: device buffer (16-byte */
/*     aligned, >= 16*t bytes) that receives the rewritten program on         */
/*     `stream` and must stay allocated and unmodified until release; the     */
/*     host `prog` may be freed on return.  BO_EINVAL if `stream` is          */
/*     capturing.  *handle receives a process-wide id (> 0).                  */
/*   bulk_execute_prepared: runs the program on mem ([p][msize] row-wise or   */
/*     [msize][p] column-wise, as bulk_execute); msize must equal the         */
/*     prepared one; stream-ordered, capturable.  BO_EINVAL on an unknown     */
/*     handle.                                                                */
/*   bulk_program_release: forgets the handle (the caller frees prog_dev).    */
/* ------------------------------------------------------------------------- */
int bulk_program_prepare(const int32_t *prog, int64_t t, int64_t msize, int nregs, void *prog_dev,
                         size_t prog_dev_bytes, void *stream, int64_t *handle);
int bulk_execute_prepared(int64_t handle, void *mem, int64_t msize, int64_t p, int dtype, int layout, void *stream);
int bulk_program_release(int64_t handle);

/* ------------------------------------------------------------------------- */
/* Compiled programs (NEXT-3).  Obliviousness makes every address of a */
/* program a constant, so the bulk execution of Theorem 2 can be  */
/* one straight-line kernel: the program unrolled, the instance memory in     */
/* registers.  The paper leaves a converter from sequential code to its bulk  */
/* CUDA program as future work; this compiles the IR above.           */
/*   bulk_program_compile: builds, with NVRTC for sm_100a (host-blocking,     */
/*     ~0.1-2 s; cached process-wide by the generated source), the kernel of  */
/*     the prepared program `handle` for one dtype and layout; afterwards     */
/*     bulk_execute_prepared with that dtype and layout launches it instead   */
/*     of the interpreter (same results bit for bit; still capturable).       */
/*     Shapes: column-wise any msize (msize <= 128: memory in registers,      */
/*     coalesced load / store of the words read / written; larger: direct     */
/*     loads grouped 32 at a time); row-wise msize <= 95 (rows staged through  */
/*     shared memory) or larger when the addresses stay in 64-word windows    */
/*     (>= 8 accesses per window; each window staged through shared memory).  */
/*     BO_EUNSUPPORTED otherwise (other row-wise programs, more               */
/*     than 200000 instructions, libnvrtc.so.12 not found: it is dlopen'ed at */
/*     the first compile, not linked) -- the interpreter keeps serving;       */
/*     BO_ECUDA with the NVRTC log if compilation fails; BO_EINVAL on an      */
/*     unknown handle or a packed layout.  Not while a stream is capturing.   */
/*   bulk_program_source: the CUDA source bulk_program_compile builds (NUL-   */
/*     terminated); *len = bytes needed incl. the NUL; copied only when       */
/*     cap >= *len.                                                           */
/* ------------------------------------------------------------------------- */
int bulk_program_compile(int64_t handle, int dtype, int layout);
int bulk_program_source(int64_t handle, int dtype, int layout, char *buf, size_t cap, size_t *len);
/*   bulk_program_generate: the same source for a HOST program (prog/t/msize/ */
/*     nregs validated as bulk_execute); no device, no handle -- for           */
/*     inspecting the generated kernel on a machine without a GPU.            */
int bulk_program_generate(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, int layout, char *buf,
                          size_t cap, size_t *len);

/* ------------------------------------------------------------------------- */
/* Layout transpose (row-wise <-> column-wise arrangement):        */
/*   dst[c*rows + r] = src[r*cols + c],  0 <= r < rows, 0 <= c < cols.        */
/* Row-wise [p][n] -> column-wise [n][p] is (rows=p, cols=n); the reverse is  */
/* (rows=n, cols=p).  elem_bytes must be 4.  Out of place: src and dst must   */
/* not overlap.  TMA-tiled when cols%4 == 0, rows%4 == 0 and both pointers    */
/* are 16-byte aligned; otherwise a padded shared-memory tile kernel.         */
/* ------------------------------------------------------------------------- */
int bulk_transpose(const void *src, void *dst, int64_t rows, int64_t cols, size_t elem_bytes,
                   void *stream);

/* ------------------------------------------------------------------------- */
/* End-to-end entry points on HOST buffers (pinned memory recommended).       */
/* The host->device copy, the computation and the device->host copy are       */
/* pipelined in chunks of instances over two internal streams; the call       */
/* returns after the result is in h_dst (it synchronises).  d_buf is a device */
/* buffer of at least bulk_*_host_bytes(...) bytes: the whole input, the      */
/* (OPT) output vector, and one workspace per internal stream (the two chunk  */
/* streams never share scratch).  h_dst may equal h_src (prefix).  Errors as  */
/* for the device entry points; a short d_buf is BO_EINVAL (message names the */
/* size needed).                                                              */
/* ------------------------------------------------------------------------- */
size_t bulk_prefix_sums_host_bytes(int64_t n, int64_t p, int dtype, int layout, int variant);
size_t bulk_triangulation_host_bytes(int64_t n, int64_t p, int dtype, int layout, int variant);
int bulk_prefix_sums_host(const void *h_src, void *h_dst, int64_t n, int64_t p, int dtype,
                          int layout, int variant, void *d_buf, size_t d_bytes, void *stream);
int bulk_triangulation_host(const void *h_c, void *h_out, int64_t n, int64_t p, int dtype,
                            int layout, int variant, void *d_buf, size_t d_bytes, void *stream);

/* ------------------------------------------------------------------------- */
/* Synthetic inputs, generated on the device by the counter-based generator  */
/* documented in bulkgen/__init__.py (same bits on host and device):         */
/*   u = mix64(seed*K_SEED + h*K_H + e*K_E), h = GLOBAL instance id h0+local. */
/* prefix kind: 0 uniform, 1 ones, 2 arange, 3 smallint.                    */
/* triangulation kind: 0 'chords' (non-negative chord weights; polygon sides, */
/*   root side and lower triangle 0 -- the configs' workload), 1 'full'        */
/*   (signed weights on every entry read, root side included; poison --       */
/*   NaN, +-inf, +-FLT_MAX, -0, garbage int32 -- on every entry never read).  */
/* ------------------------------------------------------------------------- */
int bulk_generate_prefix(void *dst, int64_t n, int64_t p, int64_t h0, uint64_t seed, int dtype,
                         int layout, int kind, void *stream);
int bulk_generate_tri(void *dst, int64_t n, int64_t p, int64_t h0, uint64_t seed, int dtype,
                      int layout, int kind, void *stream);

/* Order-independent checksum of a result (values: [p][n] row-wise, [n][p]   */
/* column-wise; n = 1 for per-instance results):                             */
/*   *acc += sum_{h,e} mix64(bits(v)*K_SEED + (h0+h)*K_H + e*K_E)  mod 2^64.  */
/* acc is a DEVICE uint64 the caller zeroes.                                 */
int bulk_checksum(const void *values, int64_t n, int64_t p, int64_t h0, int layout,
                  uint64_t *acc, void *stream);

/* ------------------------------------------------------------------------- */
/* Introspection.                                                             */
/* ------------------------------------------------------------------------- */
const char *bulk_last_error(void);       /* thread-local message, "" if none     */
/* Variant BO_AUTO resolves to for these arguments (or the forced one).       */
int bulk_prefix_sums_variant(int64_t n, int64_t p, int dtype, int layout, int variant,
                             const void *src, const void *dst);
int bulk_triangulation_variant(int64_t n, int64_t p, int dtype, int layout, int variant);
/* Number of CUDA kernels this library has launched in this process.         */
uint64_t bulk_launch_count(void);
/* Library version string. */
const char *bulk_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BULKOBL_H */
