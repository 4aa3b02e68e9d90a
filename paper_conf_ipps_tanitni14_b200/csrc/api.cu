// api.cu -- the C ABI of libbulkobl.so (include/bulkobl.h): argument
// validation, variant resolution, stream-ordered launches, and the pipelined
// host-buffer entry points.  No computation happens on the CPU.
#include "common.cuh"
#include "exec.h"
#include "jit.h"

#include <cstring>
#include <mutex>
#include <set>
#include <string>
#include <utility>
#include <map>
#include <vector>

namespace bo {

// ---------------------------------------------------------------- errors
static thread_local std::string t_err;
std::atomic<uint64_t> g_launches{0};

void set_error(const std::string &msg) { t_err = msg; }
int fail(int status, const std::string &msg) {
    set_error(msg);
    return status;
}
int cuda_check(cudaError_t e, const char *what) {
    if (e == cudaSuccess) return BO_OK;
    return fail(BO_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

int max_blocks_per_sm(const void *func, int threads, size_t smem) {
    struct Entry {
        const void *f;
        int threads, dev, blocks;
        size_t smem;
    };
    static std::mutex mu;
    static std::vector<Entry> memo;
    int dev = 0;
    cudaGetDevice(&dev);
    {
        std::lock_guard<std::mutex> lk(mu);
        for (const Entry &e : memo)
            if (e.f == func && e.threads == threads && e.smem == smem && e.dev == dev) return e.blocks;
    }
    int blocks = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, func, threads, smem) != cudaSuccess) {
        cudaGetLastError();
        blocks = 1;
    }
    std::lock_guard<std::mutex> lk(mu);
    memo.push_back(Entry{func, threads, dev, blocks, smem});
    return blocks;
}

bool ensure_dyn_smem(const void *func, int bytes) {
    // the opt-in is a per-(device, kernel) maximum: only ever raise it (a kernel
    // launched with several sizes, e.g. the executor's staged one, must not have
    // a later smaller opt-in undo an earlier larger one)
    static std::mutex mu;
    static std::map<std::pair<int, const void *>, int> set_to;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return false;
    const auto key = std::make_pair(dev, func);
    std::lock_guard<std::mutex> g(mu);
    auto it = set_to.find(key);
    if (it != set_to.end() && it->second >= bytes) return true;
    if (cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) != cudaSuccess) return false;
    set_to[key] = bytes;
    return true;
}

int work_slot_for(cudaStream_t st) {
    // A queue slot is reset by the last CTA of the launch that used it, so two
    // launches may share one only if the second cannot start before the first
    // has finished: launches on one stream (griddepcontrol.wait precedes every
    // access to the slot).  So each (device, stream) owns a slot, keyed by the
    // stream's process-unique id (cudaStreamGetId: a destroyed stream's handle
    // may be reused while its work still runs; cudaStreamPerThread resolves to
    // the calling thread's stream).  A launch being captured into a graph gets
    // none (-1: static tile striding): the graph may be replayed on any stream,
    // beside eager launches on this one.
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(st, &cap) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    if (cap != cudaStreamCaptureStatusNone) return -1;   // (cudaStreamGetId would invalidate a capture)
    unsigned long long sid = 0;
    if (cudaStreamGetId(st, &sid) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    static std::mutex mu;
    static std::vector<std::pair<int, unsigned long long>> owners;   // (device, stream id), first use order
    std::lock_guard<std::mutex> g(mu);
    int used_on_dev = 0;
    for (const auto &o : owners) {
        if (o.first != dev) continue;
        if (o.second == sid) return used_on_dev;
        ++used_on_dev;
    }
    if (used_on_dev >= kWorkSlots) return -1;                   // beyond 256 streams: static striding
    owners.emplace_back(dev, sid);
    return used_on_dev;
}

// ---------------------------------------------------------------- TMA maps
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            p = nullptr;
        return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    }();
    return fn;
}

bool make_tmap_2d(CUtensorMap *map, const void *base, uint64_t rows, uint64_t cols, uint32_t box_rows,
                  uint32_t box_cols, CUtensorMapSwizzle swz, CUtensorMapL2promotion l2) {
    // The encoded map depends only on these arguments, so a repeated call on the
    // same buffer and shape reuses it: encoding costs several microseconds of
    // host time, more than a small config's kernel (thread-local, 16 entries).
    struct Entry {
        const void *base;
        uint64_t rows, cols;
        uint32_t box_rows, box_cols;
        int swz, l2;
        CUtensorMap map;
    };
    static thread_local Entry memo[16];
    static thread_local int filled = 0, next = 0;
    for (int i = 0; i < filled; ++i) {
        const Entry &e = memo[i];
        if (e.base == base && e.rows == rows && e.cols == cols && e.box_rows == box_rows && e.box_cols == box_cols &&
            e.swz == static_cast<int>(swz) && e.l2 == static_cast<int>(l2)) {
            *map = e.map;
            return true;
        }
    }
    auto fn = encode_fn();
    if (!fn) return false;
    cuuint64_t dims[2] = {cols, rows};
    cuuint64_t strides[1] = {cols * 4};
    cuuint32_t box[2] = {box_cols, box_rows};
    cuuint32_t es[2] = {1, 1};
    CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<void *>(base), dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, swz, l2,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return false;
    memo[next] = Entry{base, rows, cols, box_rows, box_cols, static_cast<int>(swz), static_cast<int>(l2), *map};
    next = (next + 1) % 16;
    filled = filled < 16 ? filled + 1 : 16;
    return true;
}

// ---------------------------------------------------------------- internals
int launch_transpose(const void *src, void *dst, int64_t rows, int64_t cols, cudaStream_t st);
int prefix_dispatch(const void *src, void *dst, int64_t n, int64_t p, int dtype, int layout, int variant,
                    void *ws, cudaStream_t st);
int resolve_prefix_variant(int64_t n, int64_t p, int dtype, int layout, int variant, const void *src,
                           const void *dst);
int tri_dispatch(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout, int variant, void *ws,
                 cudaStream_t st);
int resolve_tri_variant(int64_t n, int64_t p, int dtype, int layout, int variant);
int launch_tri_chords(const void *c, void *out, int16_t *chords, int64_t n, int64_t p, int dtype, int layout,
                      cudaStream_t st);
size_t tri_workspace(int64_t n, int64_t p, int variant);
int launch_gen_prefix(void *, int64_t, int64_t, int64_t, uint64_t, int, int, int, cudaStream_t);
int launch_gen_tri(void *, int64_t, int64_t, int64_t, uint64_t, int, int, int, cudaStream_t);
int launch_checksum(const void *, int64_t, int64_t, int64_t, int, uint64_t *, cudaStream_t);


static constexpr int64_t kMaxElems = int64_t(1) << 40;

static bool valid_dtype(int d) { return d == BO_I32 || d == BO_F32; }
static bool valid_layout(int l) { return l == BO_ROW_WISE || l == BO_COLUMN_WISE; }
static bool valid_tri_layout(int l) { return l >= BO_ROW_WISE && l <= BO_PACKED_COLUMN; }
// weights per instance in a layout: n*n dense, (n-1)(n-2)/2 packed
static int64_t tri_words(int64_t n, int layout) { return layout >= BO_PACKED_ROW ? (n - 1) * (n - 2) / 2 : n * n; }

static bool ranges_partially_overlap(const void *a, const void *b, size_t bytes) {
    const uintptr_t x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
    if (x == y) return false;
    return x < y + bytes && y < x + bytes;
}

static bool ranges_intersect(const void *a, size_t abytes, const void *b, size_t bbytes) {
    const uintptr_t x = reinterpret_cast<uintptr_t>(a), y = reinterpret_cast<uintptr_t>(b);
    return x < y + bbytes && y < x + abytes;
}

static int check_prefix_args(const void *src, const void *dst, int64_t n, int64_t p, int dtype, int layout,
                             int variant) {
    if (n < 0 || p < 0) return fail(BO_EINVAL, "prefix: n and p must be >= 0");
    if (!valid_dtype(dtype)) return fail(BO_EINVAL, "prefix: dtype must be BO_I32 or BO_F32");
    if (!valid_layout(layout)) return fail(BO_EINVAL, "prefix: layout must be BO_ROW_WISE or BO_COLUMN_WISE");
    if (n > 0 && p > kMaxElems / n) return fail(BO_EINVAL, "prefix: n*p too large");
    if (n * p > 0 && (!src || !dst)) return fail(BO_EINVAL, "prefix: NULL pointer");
    if (n * p > 0 && ranges_partially_overlap(src, dst, static_cast<size_t>(n * p) * 4))
        return fail(BO_EINVAL, "prefix: src and dst partially overlap");
    switch (variant) {
        case BO_AUTO:
        case BO_PS_NAIVE:
            return BO_OK;
        case BO_PS_ACROSS:
            if (layout != BO_COLUMN_WISE) return fail(BO_EUNSUPPORTED, "prefix ACROSS needs the column-wise layout");
            return BO_OK;
        case BO_PS_WARPSCAN:
        case BO_PS_FUSED_ROW:
        case BO_PS_TRANSPOSED:
            if (layout != BO_ROW_WISE) return fail(BO_EUNSUPPORTED, "prefix variant needs the row-wise layout");
            return BO_OK;
        default:
            return fail(BO_EINVAL, "prefix: unknown variant");
    }
}

static int check_tri_args(const void *c, const void *out, int64_t n, int64_t p, int dtype, int layout,
                          int variant) {
    if (n < 3 || n > 4096) return fail(BO_EINVAL, "triangulation: need 3 <= n <= 4096");
    if (p < 0) return fail(BO_EINVAL, "triangulation: p must be >= 0");
    if (!valid_dtype(dtype)) return fail(BO_EINVAL, "triangulation: dtype must be BO_I32 or BO_F32");
    if (!valid_tri_layout(layout)) return fail(BO_EINVAL, "triangulation: bad layout");
    if (p > kMaxElems / (n * n)) return fail(BO_EINVAL, "triangulation: n*n*p too large");
    if (p > 0 && (!c || !out)) return fail(BO_EINVAL, "triangulation: NULL pointer");
    if (variant != BO_AUTO && (variant < BO_TRI_UMM_GLOBAL || variant > BO_TRI_TILED_GLOBAL8))
        return fail(BO_EINVAL, "triangulation: unknown variant");
    return BO_OK;
}

static size_t prefix_ws(int64_t n, int64_t p, int variant) {
    return variant == BO_PS_TRANSPOSED ? static_cast<size_t>(n) * p * 4 : 0;
}

// Internal streams for the host-buffer pipeline (one pair per device).
// `mu` is held from the ev_start record to the caller's final waits, so two
// host threads never interleave chunks on the internal streams or re-record
// ev_start between another call's record and its waits.
struct HostPipe {
    std::mutex mu;
    cudaStream_t s[2] = {nullptr, nullptr};
    cudaEvent_t ev_start = nullptr, ev_done[2] = {nullptr, nullptr};
};
static HostPipe *host_pipe() {
    static std::mutex mu;
    static std::vector<HostPipe *> pipes;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> g(mu);
    if (static_cast<int>(pipes.size()) <= dev) pipes.resize(dev + 1, nullptr);
    if (!pipes[dev]) {
        auto *hp = new HostPipe;
        for (int i = 0; i < 2; ++i) {
            cudaStreamCreateWithFlags(&hp->s[i], cudaStreamNonBlocking);
            cudaEventCreateWithFlags(&hp->ev_done[i], cudaEventDisableTiming);
        }
        cudaEventCreateWithFlags(&hp->ev_start, cudaEventDisableTiming);
        pipes[dev] = hp;
    }
    return pipes[dev];
}

#ifndef BO_HOST_CHUNKS
#define BO_HOST_CHUNKS 64     // measured: 8 -> 95.2 ms, 32 -> 89.8 ms per 8 GiB round trip (PCIe-bound);
                              // r02 A/B on one box: 16 / 32 / 64 / 128 -> 96.5 / 94.0 / 91.4 / 93.3 ms
#endif
static int64_t host_chunk(int64_t p) {
    // BO_HOST_CHUNKS chunks, multiple of 128 instances, so copies of chunk k+1
    // overlap compute/copy-back of chunk k
    int64_t ch = (p + BO_HOST_CHUNKS - 1) / BO_HOST_CHUNKS;
    ch = ((ch + 127) / 128) * 128;
    return std::max<int64_t>(std::min<int64_t>(ch, p), 1);
}

}  // namespace bo

using namespace bo;

extern "C" {

const char *bulk_last_error(void) { return t_err.c_str(); }
uint64_t bulk_launch_count(void) { return g_launches.load(); }
const char *bulk_version(void) { return "bulkobl 0.1 (sm_100a)"; }

int bulk_prefix_sums_variant(int64_t n, int64_t p, int dtype, int layout, int variant, const void *src,
                             const void *dst) {
    return resolve_prefix_variant(n, p, dtype, layout, variant, src, dst);
}

size_t bulk_prefix_sums_workspace(int64_t n, int64_t p, int dtype, int layout, int variant) {
    return prefix_ws(n, p, resolve_prefix_variant(n, p, dtype, layout, variant, nullptr, nullptr));
}

int bulk_prefix_sums(const void *src, void *dst, int64_t n, int64_t p, int dtype, int layout, int variant,
                     void *workspace, size_t workspace_bytes, void *stream) {
    t_err.clear();
    int rc = check_prefix_args(src, dst, n, p, dtype, layout, variant);
    if (rc) return rc;
    if (n * p == 0) return BO_OK;
    const int v = resolve_prefix_variant(n, p, dtype, layout, variant, src, dst);
    const size_t need = prefix_ws(n, p, v);
    if (need > 0 && (!workspace || workspace_bytes < need))
        return fail(BO_EINVAL, "prefix: workspace too small (need " + std::to_string(need) + " bytes)");
    // the workspace (need bytes) must share no byte with src or dst (n*p*4 bytes each)
    if (need > 0 && (ranges_intersect(workspace, need, src, static_cast<size_t>(n * p) * 4) ||
                     ranges_intersect(workspace, need, dst, static_cast<size_t>(n * p) * 4)))
        return fail(BO_EINVAL, "prefix: workspace overlaps the data");
    return prefix_dispatch(src, dst, n, p, dtype, layout, v, workspace, static_cast<cudaStream_t>(stream));
}

int bulk_triangulation_variant(int64_t n, int64_t p, int dtype, int layout, int variant) {
    return resolve_tri_variant(n, p, dtype, layout, variant);
}

size_t bulk_triangulation_workspace(int64_t n, int64_t p, int dtype, int layout, int variant) {
    if (n < 3 || p < 0) return 0;
    return tri_workspace(n, p, resolve_tri_variant(n, p, dtype, layout, variant));
}

int bulk_triangulation(const void *c, void *out, int64_t n, int64_t p, int dtype, int layout, int variant,
                       void *workspace, size_t workspace_bytes, void *stream) {
    t_err.clear();
    int rc = check_tri_args(c, out, n, p, dtype, layout, variant);
    if (rc) return rc;
    if (p == 0) return BO_OK;
    const int v = resolve_tri_variant(n, p, dtype, layout, variant);
    const size_t need = tri_workspace(n, p, v);
    if (need > 0 && (!workspace || workspace_bytes < need))
        return fail(BO_EINVAL, "triangulation: workspace too small (need " + std::to_string(need) + " bytes)");
    return tri_dispatch(c, out, n, p, dtype, layout, v, workspace, static_cast<cudaStream_t>(stream));
}

// Host validation of an oblivious program (bulk_execute / bulk_program_prepare):
// every register < nregs and every address < msize, so the kernel never leaves
// the instance memory.  Registers start at 0: *uninit_read tells whether some
// register is read before it is written (then the kernel zeroes its file).
static int exec_validate(const int32_t *prog, int64_t t, int64_t msize, int nregs, bool *uninit_read) {
    uint64_t written = 0;
    *uninit_read = false;
    auto use = [&](int32_t r) { if (!((written >> r) & 1)) *uninit_read = true; };
    for (int64_t i = 0; i < t; ++i) {
        const int32_t op = prog[4 * i], x = prog[4 * i + 1], y = prog[4 * i + 2], z = prog[4 * i + 3];
        auto reg = [&](int32_t r) { return r >= 0 && r < nregs; };
        auto adr = [&](int32_t a) { return a >= 0 && a < msize; };
        bool ok;
        switch (op) {
            case 0: ok = reg(x) && adr(y); break;
            case 1: ok = adr(x) && reg(y); break;
            case 2: case 3: case 4: case 5: ok = reg(x) && reg(y) && reg(z); break;
            case 6: ok = reg(x) && reg(y); break;
            case 7: ok = reg(x); break;
            default: ok = false;
        }
        if (!ok) return fail(BO_EINVAL, "execute: bad instruction " + std::to_string(i));
        switch (op) {                                      // reads, then the write
            case 1: use(y); break;
            case 2: case 3: case 4: case 5: use(y); use(z); written |= 1ull << x; break;
            case 6: use(y); written |= 1ull << x; break;
            default: written |= 1ull << x; break;      // LOAD, CONST
        }
    }
    return BO_OK;
}

static int exec_check_sizes(int64_t t, int64_t msize, int64_t p, int nregs) {
    if (t < 0 || msize < 0 || p < 0) return fail(BO_EINVAL, "execute: t, msize and p must be >= 0");
    if (nregs < 1 || nregs > 64) return fail(BO_EINVAL, "execute: need 1 <= nregs <= 64");
    if (msize > 0 && p > kMaxElems / msize) return fail(BO_EINVAL, "execute: msize*p too large");
    if (msize > INT32_MAX) return fail(BO_EINVAL, "execute: msize too large");
    return BO_OK;
}

int bulk_execute(const int32_t *prog, int64_t t, void *prog_dev, size_t prog_dev_bytes, void *mem, int64_t msize,
                 int64_t p, int dtype, int layout, int nregs, void *stream) {
    t_err.clear();
    if (int rc = exec_check_sizes(t, msize, p, nregs)) return rc;
    if (!valid_dtype(dtype) || !valid_layout(layout)) return fail(BO_EINVAL, "execute: bad dtype or layout");
    if (t == 0 || p == 0) return BO_OK;
    if (!prog || !mem) return fail(BO_EINVAL, "execute: NULL pointer");
    if (!prog_dev || prog_dev_bytes < static_cast<size_t>(t) * 16 || !aligned16(prog_dev))
        return fail(BO_EINVAL, "execute: device program buffer must be 16-byte aligned and >= 16*t bytes");
    bool uninit_read = false;
    if (int rc = exec_validate(prog, t, msize, nregs, &uninit_read)) return rc;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    // Outside graph capture the uploaded program is the fused one (exec.cu:
    // superinstructions; never longer than `prog`).  A captured copy node reads
    // its host source at every replay, so under capture the caller's own `prog`
    // is uploaded as it is (bulk_program_prepare gives a capturable fused one).
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    int rc = cuda_check(cudaStreamIsCapturing(st, &cap), "execute: stream");
    if (rc) return rc;
    ExecProgram ep{{}, 0};
    const int32_t *up = prog;
    int64_t tu = t;
    if (cap == cudaStreamCaptureStatusNone) {
        ep = exec_device_program(prog, t, msize, nregs);
        up = ep.words.data();
        tu = static_cast<int64_t>(ep.words.size() / 4);
    }
    rc = cuda_check(cudaMemcpyAsync(prog_dev, up, static_cast<size_t>(tu) * 16, cudaMemcpyHostToDevice, st),
                    "execute: program upload");
    if (rc) return rc;
    return launch_exec(prog_dev, tu, mem, msize, p, dtype, layout, nregs, uninit_read ? nregs : 0, ep.wmax, st);
}

// ---- prepared programs: validated, fused and uploaded once
namespace {
struct PreparedProgram {
    const void *dev;
    int64_t tu, msize;
    int nregs, nzero, wmax;
    const void *jit[2][2];      // compiled kernels [dtype][layout] (bulk_program_compile), or null
};
std::mutex g_prep_mu;
std::map<int64_t, PreparedProgram> g_prep;
std::map<int64_t, std::vector<int32_t>> g_prep_src;   // the validated program as given (for compiling)
int64_t g_prep_next = 1;
}  // namespace

int bulk_program_prepare(const int32_t *prog, int64_t t, int64_t msize, int nregs, void *prog_dev,
                         size_t prog_dev_bytes, void *stream, int64_t *handle) {
    t_err.clear();
    if (!handle) return fail(BO_EINVAL, "prepare: NULL handle");
    *handle = 0;
    if (int rc = exec_check_sizes(t, msize, 0, nregs)) return rc;
    if (t > 0 && !prog) return fail(BO_EINVAL, "prepare: NULL program");
    if (!prog_dev || prog_dev_bytes < static_cast<size_t>(t) * 16 || !aligned16(prog_dev))
        return fail(BO_EINVAL, "prepare: device program buffer must be 16-byte aligned and >= 16*t bytes");
    bool uninit_read = false;
    if (int rc = exec_validate(prog, t, msize, nregs, &uninit_read)) return rc;
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    int rc = cuda_check(cudaStreamIsCapturing(st, &cap), "prepare: stream");
    if (rc) return rc;
    if (cap != cudaStreamCaptureStatusNone) return fail(BO_EINVAL, "prepare: not allowed while the stream is capturing");
    const ExecProgram ep = exec_device_program(prog, t, msize, nregs);
    const std::vector<int32_t> &fused = ep.words;
    const int64_t tu = static_cast<int64_t>(fused.size() / 4);
    if (tu > 0) {
        // pageable source: the call returns once the words are staged, so the
        // temporary may go; stream-ordered before any later launch on `stream`
        rc = cuda_check(cudaMemcpyAsync(prog_dev, fused.data(), static_cast<size_t>(tu) * 16, cudaMemcpyHostToDevice, st),
                        "prepare: program upload");
        if (rc) return rc;
    }
    std::lock_guard<std::mutex> g(g_prep_mu);
    const int64_t h = g_prep_next++;
    g_prep[h] = PreparedProgram{prog_dev, tu, msize, nregs, uninit_read ? nregs : 0, ep.wmax, {{nullptr, nullptr}, {nullptr, nullptr}}};
    g_prep_src[h].assign(prog, prog + 4 * t);
    *handle = h;
    return BO_OK;
}

int bulk_execute_prepared(int64_t handle, void *mem, int64_t msize, int64_t p, int dtype, int layout, void *stream) {
    t_err.clear();
    PreparedProgram pp;
    {
        std::lock_guard<std::mutex> g(g_prep_mu);
        auto it = g_prep.find(handle);
        if (it == g_prep.end()) return fail(BO_EINVAL, "execute_prepared: unknown program handle");
        pp = it->second;
    }
    if (msize != pp.msize) return fail(BO_EINVAL, "execute_prepared: msize differs from the prepared program's");
    if (int rc = exec_check_sizes(0, msize, p, pp.nregs)) return rc;
    if (!valid_dtype(dtype) || !valid_layout(layout)) return fail(BO_EINVAL, "execute: bad dtype or layout");
    if (pp.tu == 0 || p == 0) return BO_OK;
    if (!mem) return fail(BO_EINVAL, "execute: NULL pointer");
    if ((layout == BO_ROW_WISE || layout == BO_COLUMN_WISE) && pp.jit[dtype][layout])
        return launch_jit(JitKernel{pp.jit[dtype][layout]}, mem, p, static_cast<cudaStream_t>(stream));
    return launch_exec(pp.dev, pp.tu, mem, msize, p, dtype, layout, pp.nregs, pp.nzero, pp.wmax,
                       static_cast<cudaStream_t>(stream));
}

int bulk_program_release(int64_t handle) {
    t_err.clear();
    std::lock_guard<std::mutex> g(g_prep_mu);
    if (g_prep.erase(handle) == 0) return fail(BO_EINVAL, "release: unknown program handle");
    g_prep_src.erase(handle);
    return BO_OK;
}

int bulk_program_compile(int64_t handle, int dtype, int layout) {
    t_err.clear();
    if (!valid_dtype(dtype) || (layout != BO_ROW_WISE && layout != BO_COLUMN_WISE))
        return fail(BO_EINVAL, "compile: dtype BO_I32 / BO_F32, layout BO_ROW_WISE / BO_COLUMN_WISE");
    std::vector<int32_t> src;
    PreparedProgram pp;
    {
        std::lock_guard<std::mutex> g(g_prep_mu);
        auto it = g_prep.find(handle);
        if (it == g_prep.end()) return fail(BO_EINVAL, "compile: unknown program handle");
        pp = it->second;
        src = g_prep_src[handle];
    }
    if (pp.jit[dtype][layout]) return BO_OK;
    JitKernel k;
    const int64_t t = static_cast<int64_t>(src.size() / 4);
    if (int rc = jit_compile(src.data(), t, pp.msize, pp.nregs, dtype, layout, &k)) return rc;
    std::lock_guard<std::mutex> g(g_prep_mu);
    auto it = g_prep.find(handle);
    if (it == g_prep.end()) return fail(BO_EINVAL, "compile: program released while compiling");
    it->second.jit[dtype][layout] = k.kernel;
    return BO_OK;
}

int bulk_program_source(int64_t handle, int dtype, int layout, char *buf, size_t cap, size_t *len) {
    t_err.clear();
    if (!len) return fail(BO_EINVAL, "program source: NULL len");
    std::vector<int32_t> src;
    PreparedProgram pp;
    {
        std::lock_guard<std::mutex> g(g_prep_mu);
        auto it = g_prep.find(handle);
        if (it == g_prep.end()) return fail(BO_EINVAL, "program source: unknown program handle");
        pp = it->second;
        src = g_prep_src[handle];
    }
    if (!valid_dtype(dtype)) return fail(BO_EINVAL, "program source: bad dtype");
    const std::string s = jit_source(src.data(), static_cast<int64_t>(src.size() / 4), pp.msize, pp.nregs, dtype, layout);
    if (s.empty()) return fail(BO_EUNSUPPORTED, "program source: this arrangement is not compiled");
    *len = s.size() + 1;
    if (buf && cap >= s.size() + 1) std::memcpy(buf, s.c_str(), s.size() + 1);
    return BO_OK;
}

int bulk_program_generate(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, int layout, char *buf,
                          size_t cap, size_t *len) {
    t_err.clear();
    if (!len) return fail(BO_EINVAL, "program generate: NULL len");
    if (int rc = exec_check_sizes(t, msize, 0, nregs)) return rc;
    if (t > 0 && !prog) return fail(BO_EINVAL, "program generate: NULL program");
    if (!valid_dtype(dtype)) return fail(BO_EINVAL, "program generate: bad dtype");
    bool uninit_read = false;
    if (int rc = exec_validate(prog, t, msize, nregs, &uninit_read)) return rc;
    const std::string s = jit_source(prog, t, msize, nregs, dtype, layout);
    if (s.empty()) return fail(BO_EUNSUPPORTED, "program generate: this arrangement is not compiled");
    *len = s.size() + 1;
    if (buf && cap >= s.size() + 1) std::memcpy(buf, s.c_str(), s.size() + 1);
    return BO_OK;
}

int bulk_triangulation_chords(const void *c, void *out, int16_t *chords, int64_t n, int64_t p, int dtype,
                              int layout, void *stream) {
    t_err.clear();
    int rc = check_tri_args(c, out, n, p, dtype, layout, BO_AUTO);
    if (rc) return rc;
    if (n > 64) return fail(BO_EUNSUPPORTED, "triangulation chords: n <= 64 (the table must fit in shared memory)");
    if (p == 0) return BO_OK;
    if (n > 3 && !chords) return fail(BO_EINVAL, "triangulation chords: NULL chords pointer");
    return launch_tri_chords(c, out, chords, n, p, dtype, layout, static_cast<cudaStream_t>(stream));
}

int bulk_transpose(const void *src, void *dst, int64_t rows, int64_t cols, size_t elem_bytes, void *stream) {
    t_err.clear();
    if (elem_bytes != 4) return fail(BO_EUNSUPPORTED, "transpose: only 4-byte elements");
    if (rows < 0 || cols < 0) return fail(BO_EINVAL, "transpose: rows and cols must be >= 0");
    if (rows > 0 && cols > kMaxElems / rows) return fail(BO_EINVAL, "transpose: rows*cols too large");
    if (rows * cols == 0) return BO_OK;
    if (!src || !dst) return fail(BO_EINVAL, "transpose: NULL pointer");
    if (src == dst || ranges_partially_overlap(src, dst, static_cast<size_t>(rows * cols) * 4))
        return fail(BO_EINVAL, "transpose: src and dst overlap (out of place only)");
    return launch_transpose(src, dst, rows, cols, static_cast<cudaStream_t>(stream));
}

int bulk_generate_prefix(void *dst, int64_t n, int64_t p, int64_t h0, uint64_t seed, int dtype, int layout,
                         int kind, void *stream) {
    t_err.clear();
    if (n < 0 || p < 0 || h0 < 0 || !valid_dtype(dtype) || !valid_layout(layout) || kind < 0 || kind > 3)
        return fail(BO_EINVAL, "generate_prefix: bad argument");
    if (n * p > 0 && !dst) return fail(BO_EINVAL, "generate_prefix: NULL pointer");
    return launch_gen_prefix(dst, n, p, h0, seed, dtype, layout, kind, static_cast<cudaStream_t>(stream));
}

int bulk_generate_tri(void *dst, int64_t n, int64_t p, int64_t h0, uint64_t seed, int dtype, int layout,
                      int kind, void *stream) {
    t_err.clear();
    if (n < 1 || p < 0 || h0 < 0 || !valid_dtype(dtype) || !valid_tri_layout(layout) || kind < 0 || kind > 1 ||
        (layout >= BO_PACKED_ROW && n < 3))
        return fail(BO_EINVAL, "generate_tri: bad argument");
    if (p > 0 && !dst) return fail(BO_EINVAL, "generate_tri: NULL pointer");
    return launch_gen_tri(dst, n, p, h0, seed, dtype, layout, kind, static_cast<cudaStream_t>(stream));
}

int bulk_checksum(const void *values, int64_t n, int64_t p, int64_t h0, int layout, uint64_t *acc, void *stream) {
    t_err.clear();
    if (n < 0 || p < 0 || h0 < 0 || !valid_layout(layout) || !acc) return fail(BO_EINVAL, "checksum: bad argument");
    if (n * p > 0 && !values) return fail(BO_EINVAL, "checksum: NULL pointer");
    return launch_checksum(values, n, p, h0, layout, acc, static_cast<cudaStream_t>(stream));
}

// ------------------------------------------------------------------ host e2e
size_t bulk_prefix_sums_host_bytes(int64_t n, int64_t p, int dtype, int layout, int variant) {
    if (n < 0 || p < 0 || n * p == 0) return 0;
    const int v = resolve_prefix_variant(n, p, dtype, layout, variant, nullptr, nullptr);
    return static_cast<size_t>(n) * p * 4 + 2 * prefix_ws(n, host_chunk(p), v);
}

int bulk_prefix_sums_host(const void *h_src, void *h_dst, int64_t n, int64_t p, int dtype, int layout,
                          int variant, void *d_buf, size_t d_bytes, void *stream) {
    t_err.clear();
    int rc = check_prefix_args(h_src, h_dst, n, p, dtype, layout, variant);
    if (rc) return rc;
    if (n * p == 0) return BO_OK;
    const int v = resolve_prefix_variant(n, p, dtype, layout, variant, nullptr, nullptr);
    const int64_t ch = host_chunk(p);
    const size_t data_bytes = static_cast<size_t>(n) * p * 4;
    const size_t ws_chunk = prefix_ws(n, ch, v);
    if (!d_buf || d_bytes < data_bytes + 2 * ws_chunk)
        return fail(BO_EINVAL, "prefix_host: device buffer too small (need " +
                                   std::to_string(data_bytes + 2 * ws_chunk) + " bytes)");
    HostPipe *hp = host_pipe();
    cudaStream_t caller = static_cast<cudaStream_t>(stream);
    std::unique_lock<std::mutex> pipe_lock(hp->mu);
    if ((rc = cuda_check(cudaEventRecord(hp->ev_start, caller), "prefix_host: event"))) return rc;
    for (int i = 0; i < 2; ++i)
        if ((rc = cuda_check(cudaStreamWaitEvent(hp->s[i], hp->ev_start, 0), "prefix_host: wait"))) return rc;
    const char *hs = static_cast<const char *>(h_src);
    char *hd = static_cast<char *>(h_dst);
    char *db = static_cast<char *>(d_buf);
    int k = 0;
    for (int64_t p0 = 0; p0 < p; p0 += ch, ++k) {
        const int64_t pc = std::min(ch, p - p0);
        cudaStream_t s = hp->s[k & 1];
        char *dchunk = db + static_cast<size_t>(p0) * n * 4;        // compact chunk, same layout
        void *ws = ws_chunk ? db + data_bytes + (k & 1) * ws_chunk : nullptr;
        if (layout == BO_ROW_WISE) {
            rc = cuda_check(cudaMemcpyAsync(dchunk, hs + static_cast<size_t>(p0) * n * 4,
                                            static_cast<size_t>(pc) * n * 4, cudaMemcpyHostToDevice, s),
                            "prefix_host: H2D");
        } else {
            rc = cuda_check(cudaMemcpy2DAsync(dchunk, pc * 4, hs + p0 * 4, p * 4, pc * 4, n, cudaMemcpyHostToDevice, s),
                            "prefix_host: H2D");
        }
        if (rc) return rc;
        if ((rc = prefix_dispatch(dchunk, dchunk, n, pc, dtype, layout, v, ws, s))) return rc;
        if (layout == BO_ROW_WISE) {
            rc = cuda_check(cudaMemcpyAsync(hd + static_cast<size_t>(p0) * n * 4, dchunk,
                                            static_cast<size_t>(pc) * n * 4, cudaMemcpyDeviceToHost, s),
                            "prefix_host: D2H");
        } else {
            rc = cuda_check(cudaMemcpy2DAsync(hd + p0 * 4, p * 4, dchunk, pc * 4, pc * 4, n, cudaMemcpyDeviceToHost, s),
                            "prefix_host: D2H");
        }
        if (rc) return rc;
    }
    for (int i = 0; i < 2; ++i) {
        if ((rc = cuda_check(cudaEventRecord(hp->ev_done[i], hp->s[i]), "prefix_host: event"))) return rc;
        if ((rc = cuda_check(cudaStreamWaitEvent(caller, hp->ev_done[i], 0), "prefix_host: wait"))) return rc;
    }
    pipe_lock.unlock();
    return cuda_check(cudaStreamSynchronize(caller), "prefix_host: sync");
}

// Scratch of one chunk stream: the UMM variant keeps a table per instance, so
// the chunks use disjoint slices of one p-sized workspace; TILED_GLOBAL keeps
// a table per CTA, so each of the two streams gets its own chunk-sized copy.
static size_t tri_host_ws(int64_t n, int64_t p, int v) {
    if (v == BO_TRI_TILED_GLOBAL || v == BO_TRI_TILED_GLOBAL8) return 2 * tri_workspace(n, host_chunk(p), v);
    return tri_workspace(n, p, v);
}

size_t bulk_triangulation_host_bytes(int64_t n, int64_t p, int dtype, int layout, int variant) {
    if (n < 3 || p <= 0 || !valid_tri_layout(layout)) return 0;
    const int v = resolve_tri_variant(n, p, dtype, layout, variant);
    const size_t ws_off = (static_cast<size_t>(tri_words(n, layout)) * p * 4 + static_cast<size_t>(p) * 4 + 255) & ~size_t(255);
    return ws_off + tri_host_ws(n, p, v);
}

int bulk_triangulation_host(const void *h_c, void *h_out, int64_t n, int64_t p, int dtype, int layout,
                            int variant, void *d_buf, size_t d_bytes, void *stream) {
    t_err.clear();
    int rc = check_tri_args(h_c, h_out, n, p, dtype, layout, variant);
    if (rc) return rc;
    if (p == 0) return BO_OK;
    const int v = resolve_tri_variant(n, p, dtype, layout, variant);
    const int64_t ch = host_chunk(p);
    const size_t nn = static_cast<size_t>(tri_words(n, layout));     // weights per instance
    const size_t c_bytes = nn * p * 4, out_bytes = static_cast<size_t>(p) * 4;
    const size_t ws_bytes = tri_host_ws(n, p, v);
    const size_t ws_off = (c_bytes + out_bytes + 255) & ~size_t(255);   // workspace 256-byte aligned
    if (!d_buf || d_bytes < ws_off + ws_bytes)
        return fail(BO_EINVAL, "triangulation_host: device buffer too small (need " +
                                   std::to_string(ws_off + ws_bytes) + " bytes)");
    HostPipe *hp = host_pipe();
    cudaStream_t caller = static_cast<cudaStream_t>(stream);
    std::unique_lock<std::mutex> pipe_lock(hp->mu);
    if ((rc = cuda_check(cudaEventRecord(hp->ev_start, caller), "tri_host: event"))) return rc;
    for (int i = 0; i < 2; ++i)
        if ((rc = cuda_check(cudaStreamWaitEvent(hp->s[i], hp->ev_start, 0), "tri_host: wait"))) return rc;
    const char *hc = static_cast<const char *>(h_c);
    char *ho = static_cast<char *>(h_out);
    char *db = static_cast<char *>(d_buf);
    char *dout = db + c_bytes;
    char *dws = db + ws_off;
    int k = 0;
    for (int64_t p0 = 0; p0 < p; p0 += ch, ++k) {
        const int64_t pc = std::min(ch, p - p0);
        cudaStream_t s = hp->s[k & 1];
        char *dchunk = db + static_cast<size_t>(p0) * nn * 4;
        if (layout == BO_ROW_WISE || layout == BO_PACKED_ROW)
            rc = cuda_check(cudaMemcpyAsync(dchunk, hc + static_cast<size_t>(p0) * nn * 4, pc * nn * 4,
                                            cudaMemcpyHostToDevice, s),
                            "tri_host: H2D");
        else
            rc = cuda_check(cudaMemcpy2DAsync(dchunk, pc * 4, hc + p0 * 4, p * 4, pc * 4, nn, cudaMemcpyHostToDevice, s),
                            "tri_host: H2D");
        if (rc) return rc;
        void *ws = nullptr;
        if (v == BO_TRI_UMM_GLOBAL) ws = dws + static_cast<size_t>(p0) * (n - 1) * (n - 1) * 4;
        else if (ws_bytes) ws = dws + (k & 1) * (ws_bytes / 2);
        if ((rc = tri_dispatch(dchunk, dout + p0 * 4, n, pc, dtype, layout, v, ws, s))) return rc;
        if ((rc = cuda_check(cudaMemcpyAsync(ho + p0 * 4, dout + p0 * 4, pc * 4, cudaMemcpyDeviceToHost, s),
                             "tri_host: D2H")))
            return rc;
    }
    for (int i = 0; i < 2; ++i) {
        if ((rc = cuda_check(cudaEventRecord(hp->ev_done[i], hp->s[i]), "tri_host: event"))) return rc;
        if ((rc = cuda_check(cudaStreamWaitEvent(caller, hp->ev_done[i], 0), "tri_host: wait"))) return rc;
    }
    pipe_lock.unlock();
    return cuda_check(cudaStreamSynchronize(caller), "tri_host: sync");
}

}  // extern "C"
