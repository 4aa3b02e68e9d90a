// jit.cu -- compiled oblivious programs (NEXT-3): a prepared program (api.cu)
// turned into one straight-line sm_100a kernel with NVRTC, so each instance
// runs the program as plain instructions on registers instead of through the
// interpreter's fetch / decode loop (exec.cu).
//
// Obliviousness (the address of step i is a(i) whatever the input) is
// what makes this possible: every address is a compile-time constant, so the
// instance memory can live in registers and the kernel is the sequential
// algorithm itself, unrolled -- the "bulk execution" of Theorem 2
// with the program known when the kernel is built.  The paper leaves a
// compiler from sequential code to its bulk CUDA program as future work
// (P:264); this compiles the library's own straight-line IR (bulkobl.h).
//
// Three shapes, chosen from the program and the arrangement:
//   R-column  msize <= 128, column-wise: thread j keeps words b[a] in
//             registers m<a>, loading (coalesced, a*p + j) the words whose first
//             access is a LOAD and storing the words the program STOREs;
//   R-row     msize <= 95, row-wise: a CTA stages its 128 instances'
//             rows through shared memory (coalesced copies, pitch msize+1),
//             then the same register program per thread;
//   S-column  larger msize, column-wise: every LOAD / STORE goes to global
//             memory at a*p + j, and the loads of each block of <= 32 LOADs are
//             issued together ahead of the block (a LOAD of an address STOREd
//             earlier in the block takes the stored value), so each thread keeps
//             up to 32 loads in flight instead of one dependent load per step.
//   W-row     larger msize, row-wise: the program cut into segments whose
//             addresses span <= 64 words; per segment the CTA's 128 rows' window
//             is staged through shared memory (coalesced), the segment runs on it
//             and it is written back if stored to -- when the windows are reused
//             (>= 8 accesses per segment on average, <= 1024 segments); other
//             row-wise programs are not compiled (the interpreter serves them).
//
// Semantics are the header's, instruction by instruction: registers start at
// 0; int32 ADD / SUB wrap mod 2^32 (done in uint32); fp32 ADD / SUB are
// __fadd_rn / __fsub_rn (no contraction); MIN r <- (r[z] < r[y] ? r[z] : r[y])
// and MAX r <- (r[y] < r[z] ? r[z] : r[y]) written exactly so (not fminf /
// fmaxf, which differ on NaN and signed zeros); CONST is a bit pattern (fp32
// constants pass through a runtime zero so ptxas cannot fold them: it rounds
// folded add.rn.f32 of immediates wrongly, see op_expr).
#include "common.cuh"
#include "jit.h"

#include <dlfcn.h>
#include <nvrtc.h>

#include <algorithm>
#include <climits>
#include <functional>
#include <map>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

namespace bo {
namespace {

constexpr int kJitThreads = 128;
#ifndef BO_JIT_MINB
#define BO_JIT_MINB 4   // bitonic n=64 column-wise: 1 (254 regs) 0.210, 4 (128) 0.205, 6 (80) 0.315, 8 (64) 0.376 ms
#endif
#ifndef BO_JIT_CAP_MSIZE
#define BO_JIT_CAP_MSIZE 64
#endif
#ifndef BO_JIT_GROUP
#define BO_JIT_GROUP 32   // measured (prefix program n=1024, p=2^20): 8 1.505, 16 1.482, 32 1.395, 64 1.568 ms
#endif
constexpr int kStreamGroup = BO_JIT_GROUP;        // LOADs issued ahead per block (streaming shape)
constexpr int64_t kMaxJitInstructions = 200000;   // NVRTC time grows with the program (~1 s at 20K)

enum Shape { kRegColumn, kRegRow, kStreamColumn, kWinRow, kNone };

bool win_row_ok(const int32_t *prog, int64_t t);
Shape jit_shape(const int32_t *prog, int64_t t, int64_t msize, int layout) {
    if (layout == BO_COLUMN_WISE) return msize <= 128 ? kRegColumn : kStreamColumn;
    if (layout == BO_ROW_WISE && msize <= 95) return kRegRow;   // 128 x 96 x 4 B = 48 KB static smem
    if (layout == BO_ROW_WISE && win_row_ok(prog, t)) return kWinRow;
    return kNone;
}

std::string op_expr(int32_t op, int32_t x, int32_t y, int32_t z, bool f32) {
    std::ostringstream s;
    const std::string rx = "r" + std::to_string(x), ry = "r" + std::to_string(y), rz = "r" + std::to_string(z);
    switch (op) {
        case 2: s << rx << " = " << (f32 ? "__fadd_rn(" + ry + ", " + rz + ")" : "(int)((unsigned)" + ry + " + (unsigned)" + rz + ")"); break;
        case 3: s << rx << " = " << (f32 ? "__fsub_rn(" + ry + ", " + rz + ")" : "(int)((unsigned)" + ry + " - (unsigned)" + rz + ")"); break;
        case 4: s << rx << " = (" << rz << " < " << ry << ") ? " << rz << " : " << ry; break;
        case 5: s << rx << " = (" << ry << " < " << rz << ") ? " << rz << " : " << ry; break;
        case 6: s << rx << " = " << ry; break;
        case 7:
            // through the runtime zero `z`: ptxas (12.9, sm_100a) constant-folds add.rn.f32 of two
            // immediates with a wrong rounding (-1.029471f + 3.4000282f folded to 0x4017b735, RN is
            // 0x4017b736), so float constants must not be visible to it
            if (f32) s << rx << " = __int_as_float(" << y << " ^ z)";
            else s << rx << " = (int)" << y;
            break;
    }
    s << ";\n";
    return s.str();
}

// Windowed row-wise shape: cut the program greedily into segments whose memory
// addresses span <= kWin words.
constexpr int kWin = 64;
#ifndef BO_JIT_WIN_UNROLL
#define BO_JIT_WIN_UNROLL 8   // window copies (prefix program row-wise): 8 1.82, 16 1.90, 32 2.59, 64 6.23 ms
#endif
struct Segment {
    int64_t i, e;
    int32_t lo, len;
    bool stores;
};
std::vector<Segment> win_segments(const int32_t *prog, int64_t t) {
    std::vector<Segment> seg;
    int64_t i = 0;
    while (i < t) {
        int64_t e = i;
        int32_t lo = INT32_MAX, hi = -1;
        bool stores = false;
        for (; e < t; ++e) {
            const int32_t op = prog[4 * e];
            if (op != 0 && op != 1) continue;
            const int32_t a = op == 0 ? prog[4 * e + 2] : prog[4 * e + 1];
            const int32_t nlo = std::min(lo, a), nhi = std::max(hi, a);
            if (nhi - nlo + 1 > kWin) break;
            lo = nlo, hi = nhi;
            stores |= op == 1;
        }
        if (hi < 0) lo = 0, hi = 0;                  // registers only
        seg.push_back({i, e, lo, hi - lo + 1, stores});
        i = e;
    }
    return seg;
}
// worth compiling only when the windows are reused: >= 8 memory accesses per segment on
// average (the interpreter's windowing rule) and a bounded number of segments (each one
// is two staged copies in the generated code)
bool win_row_ok(const int32_t *prog, int64_t t) {
    int64_t mem = 0;
    for (int64_t i = 0; i < t; ++i) mem += prog[4 * i] == 0 || prog[4 * i] == 1;
    const auto seg = win_segments(prog, t);
    return seg.size() <= 1024 && mem >= 8 * static_cast<int64_t>(seg.size());
}

std::string generate(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, Shape shape) {
    const bool f32 = dtype == BO_F32;
    std::ostringstream s;
    s << "// generated by libbulkobl (jit.cu): " << t << " instructions, msize " << msize << "\n";
    s << "typedef " << (f32 ? "float" : "int") << " T;\n";
    // register shapes: cap the registers so >= 4 CTAs (16 warps) fit per SM when the memory is small
    // (uncapped, nvcc keeps all 64 loaded words of the bitonic sort live at 254 registers: 8 warps / SM)
    const int minb = (shape != kStreamColumn && msize <= BO_JIT_CAP_MSIZE) ? BO_JIT_MINB : 1;
    s << "extern \"C\" __global__ void __launch_bounds__(" << kJitThreads << ", " << minb
      << ") bo_prog(T *__restrict__ mem, long long p, int z) {\n";
    s << "  asm volatile(\"griddepcontrol.wait;\" ::: \"memory\");\n";
    s << "  T";
    for (int r = 0; r < nregs; ++r) s << (r ? ", " : " ") << "r" << r << " = (T)0";
    s << ";\n";
    if (shape == kRegColumn || shape == kRegRow) {
        std::vector<int> first(msize, -1);   // -1 untouched, 0 first access LOAD, 1 first access STORE
        std::vector<char> written(msize, 0);
        for (int64_t i = 0; i < t; ++i) {
            const int32_t op = prog[4 * i], x = prog[4 * i + 1], y = prog[4 * i + 2];
            if (op == 0 && first[y] < 0) first[y] = 0;
            if (op == 1) {
                if (first[x] < 0) first[x] = 1;
                written[x] = 1;
            }
        }
        if (shape == kRegColumn) {
            s << "  const long long j = (long long)blockIdx.x * " << kJitThreads << " + threadIdx.x;\n";
            s << "  if (j >= p) return;\n";
            s << "  T *__restrict__ b = mem + j;\n";
            for (int64_t a = 0; a < msize; ++a)
                if (first[a] >= 0) s << "  T m" << a << (first[a] == 0 ? " = b[" + std::to_string(a) + "LL * p]" : "") << ";\n";
        } else {
            s << "  __shared__ T tile[" << kJitThreads * (msize + 1) << "];\n";
            s << "  const long long j0 = (long long)blockIdx.x * " << kJitThreads << ";\n";
            s << "  const int cnt = (int)(p - j0 < " << kJitThreads << " ? p - j0 : " << kJitThreads << ");\n";
            s << "  T *__restrict__ g = mem + j0 * " << msize << "LL;\n";
            s << "  for (int i = threadIdx.x; i < cnt * " << msize << "; i += " << kJitThreads << ") { const int q = i / "
              << msize << ", a = i - q * " << msize << "; tile[q * " << msize + 1 << " + a] = g[i]; }\n";
            s << "  __syncthreads();\n";
            s << "  if (threadIdx.x < cnt) {\n";
            s << "  T *sr = tile + threadIdx.x * " << msize + 1 << ";\n";
            for (int64_t a = 0; a < msize; ++a)
                if (first[a] >= 0) s << "  T m" << a << (first[a] == 0 ? " = sr[" + std::to_string(a) + "]" : "") << ";\n";
        }
        for (int64_t i = 0; i < t; ++i) {
            const int32_t op = prog[4 * i], x = prog[4 * i + 1], y = prog[4 * i + 2], z = prog[4 * i + 3];
            if (op == 0) s << "  r" << x << " = m" << y << ";\n";
            else if (op == 1) s << "  m" << x << " = r" << y << ";\n";
            else s << "  " << op_expr(op, x, y, z, f32);
        }
        if (shape == kRegColumn) {
            for (int64_t a = 0; a < msize; ++a)
                if (written[a]) s << "  b[" << a << "LL * p] = m" << a << ";\n";
        } else {
            bool any = false;
            for (int64_t a = 0; a < msize; ++a)
                if (written[a]) s << "  sr[" << a << "] = m" << a << ";\n", any = true;
            s << "  }\n";
            if (any) {
                s << "  __syncthreads();\n";
                s << "  for (int i = threadIdx.x; i < cnt * " << msize << "; i += " << kJitThreads << ") { const int q = i / "
                  << msize << ", a = i - q * " << msize << "; g[i] = tile[q * " << msize + 1 << " + a]; }\n";
            }
        }
    } else if (shape == kWinRow) {
        // row-wise, larger memories: the program in segments whose addresses span <= kWin
        // words; per segment the CTA's 128 rows' window [lo, lo+len) is staged through shared
        // memory (coalesced: consecutive threads take consecutive words of a row), the
        // segment runs on it, and it is written back when the segment stored into it
        s << "  __shared__ T tile[" << kJitThreads * (kWin + 1) << "];\n";
        s << "  const long long j0 = (long long)blockIdx.x * " << kJitThreads << ";\n";
        s << "  const int cnt = (int)(p - j0 < " << kJitThreads << " ? p - j0 : " << kJitThreads << ");\n";
        s << "  T *__restrict__ g = mem + j0 * " << msize << "LL;\n";
        s << "  T *sr = tile + threadIdx.x * " << kWin + 1 << ";\n";
        bool first_seg = true;
        for (const Segment &g : win_segments(prog, t)) {
            const int32_t lo = g.lo, len = g.len;
            if (!first_seg) s << "  __syncthreads();\n";
            first_seg = false;
            s << "#pragma unroll " << BO_JIT_WIN_UNROLL << "\n  for (int i = threadIdx.x; i < cnt * " << len << "; i += " << kJitThreads
              << ") { const int q = i / " << len << ", a = i - q * " << len << "; tile[q * " << kWin + 1
              << " + a] = g[(long long)q * " << msize << "LL + " << lo << " + a]; }\n";
            s << "  __syncthreads();\n  if (threadIdx.x < cnt) {\n";
            for (int64_t k = g.i; k < g.e; ++k) {
                const int32_t op = prog[4 * k], x = prog[4 * k + 1], y = prog[4 * k + 2], z = prog[4 * k + 3];
                if (op == 0) s << "  r" << x << " = sr[" << y - lo << "];\n";
                else if (op == 1) s << "  sr[" << x - lo << "] = r" << y << ";\n";
                else s << "  " << op_expr(op, x, y, z, f32);
            }
            s << "  }\n";
            if (g.stores) {
                s << "  __syncthreads();\n";
                s << "#pragma unroll " << BO_JIT_WIN_UNROLL << "\n  for (int i = threadIdx.x; i < cnt * " << len << "; i += " << kJitThreads
                  << ") { const int q = i / " << len << ", a = i - q * " << len << "; g[(long long)q * " << msize
                  << "LL + " << lo << " + a] = tile[q * " << kWin + 1 << " + a]; }\n";
            }
        }
    } else {   // kStreamColumn
        // loads / stores as inline PTX: opaque to NVVM, whose alias analysis over thousands
        // of b + a*p accesses is what made this shape slow to compile (~90 s at 3K
        // instructions), and issued in exactly the order emitted here
        s << "  const long long j = (long long)blockIdx.x * " << kJitThreads << " + threadIdx.x;\n";
        s << "  if (j >= p) return;\n";
        s << "  T *__restrict__ b = mem + j;\n";
        s << "  const long long ps = p * " << (f32 ? 4 : 4) << "LL;\n";
        if (f32) {
            s << "#define LDG(v, a) asm volatile(\"ld.global.f32 %0, [%1];\" : \"=f\"(v) : \"l\"((const char *)b + (a) * ps) : \"memory\")\n";
            s << "#define STG(a, v) asm volatile(\"st.global.f32 [%0], %1;\" :: \"l\"((char *)b + (a) * ps), \"f\"(v) : \"memory\")\n";
        } else {
            s << "#define LDG(v, a) asm volatile(\"ld.global.b32 %0, [%1];\" : \"=r\"(v) : \"l\"((const char *)b + (a) * ps) : \"memory\")\n";
            s << "#define STG(a, v) asm volatile(\"st.global.b32 [%0], %1;\" :: \"l\"((char *)b + (a) * ps), \"r\"(v) : \"memory\")\n";
        }
        int64_t i = 0, tmp = 0;
        while (i < t) {
            // a block: up to kStreamGroup LOADs (and at most 4x as many instructions)
            int64_t e = i, nload = 0;
            while (e < t && nload < kStreamGroup && e - i < 4 * kStreamGroup) nload += prog[4 * e] == 0, ++e;
            std::map<int32_t, std::string> fwd;       // address -> value STOREd earlier in the block
            std::map<int64_t, std::string> hoisted;   // instruction -> its hoisted load temp
            {
                std::map<int32_t, bool> stored;
                for (int64_t k = i; k < e; ++k) {
                    const int32_t op = prog[4 * k], x = prog[4 * k + 1], y = prog[4 * k + 2];
                    if (op == 0 && !stored.count(y)) {
                        const std::string v = "l" + std::to_string(tmp++);
                        s << "  T " << v << "; LDG(" << v << ", " << y << ");\n";
                        hoisted[k] = v;
                    }
                    if (op == 1) stored[x] = true;
                }
            }
            for (int64_t k = i; k < e; ++k) {
                const int32_t op = prog[4 * k], x = prog[4 * k + 1], y = prog[4 * k + 2], z = prog[4 * k + 3];
                if (op == 0) {
                    auto h = hoisted.find(k);
                    s << "  r" << x << " = " << (h != hoisted.end() ? h->second : fwd.at(y)) << ";\n";
                } else if (op == 1) {
                    const std::string v = "f" + std::to_string(tmp++);
                    s << "  const T " << v << " = r" << y << "; STG(" << x << ", " << v << ");\n";
                    fwd[x] = v;
                } else {
                    s << "  " << op_expr(op, x, y, z, f32);
                }
            }
            i = e;
        }
    }
    s << "}\n";
    return s.str();
}

struct Compiled {
    cudaLibrary_t lib;
    cudaKernel_t kern;
};
std::mutex g_mu;
std::map<size_t, std::vector<std::pair<std::string, Compiled>>> g_cache;   // source hash -> (source, kernel)

// NVRTC is opened at the first compile (dlopen), not linked: the rest of the
// library loads and runs without it, and a process that already loaded a
// libnvrtc.so.12 (torch does) shares that one.
struct Nvrtc {
    decltype(&nvrtcCreateProgram) create;
    decltype(&nvrtcCompileProgram) compile;
    decltype(&nvrtcGetProgramLogSize) log_size;
    decltype(&nvrtcGetProgramLog) log;
    decltype(&nvrtcGetCUBINSize) cubin_size;
    decltype(&nvrtcGetCUBIN) cubin;
    decltype(&nvrtcDestroyProgram) destroy;
    decltype(&nvrtcGetErrorString) error;
    bool ok;
};
const Nvrtc &nvrtc() {
    static const Nvrtc api = [] {
        Nvrtc a{};
        void *h = dlopen("libnvrtc.so.12", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("/usr/local/cuda/lib64/libnvrtc.so.12", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return a;
        a.create = reinterpret_cast<decltype(a.create)>(dlsym(h, "nvrtcCreateProgram"));
        a.compile = reinterpret_cast<decltype(a.compile)>(dlsym(h, "nvrtcCompileProgram"));
        a.log_size = reinterpret_cast<decltype(a.log_size)>(dlsym(h, "nvrtcGetProgramLogSize"));
        a.log = reinterpret_cast<decltype(a.log)>(dlsym(h, "nvrtcGetProgramLog"));
        a.cubin_size = reinterpret_cast<decltype(a.cubin_size)>(dlsym(h, "nvrtcGetCUBINSize"));
        a.cubin = reinterpret_cast<decltype(a.cubin)>(dlsym(h, "nvrtcGetCUBIN"));
        a.destroy = reinterpret_cast<decltype(a.destroy)>(dlsym(h, "nvrtcDestroyProgram"));
        a.error = reinterpret_cast<decltype(a.error)>(dlsym(h, "nvrtcGetErrorString"));
        a.ok = a.create && a.compile && a.log_size && a.log && a.cubin_size && a.cubin && a.destroy && a.error;
        return a;
    }();
    return api;
}

int nvrtc_fail(nvrtcResult r, const char *what, const std::string &log = "") {
    return fail(BO_ECUDA, std::string("program compile: ") + what + ": " + nvrtc().error(r) +
                              (log.empty() ? "" : "\n" + log.substr(0, 2000)));
}

int compile_source(const std::string &src, Compiled *out) {
    const Nvrtc &N = nvrtc();
    if (!N.ok) return fail(BO_EUNSUPPORTED, "program compile: libnvrtc.so.12 not found (the interpreter keeps serving)");
    nvrtcProgram prog;
    nvrtcResult r = N.create(&prog, src.c_str(), "bo_prog.cu", 0, nullptr, nullptr);
    if (r != NVRTC_SUCCESS) return nvrtc_fail(r, "nvrtcCreateProgram");
    const char *opts[] = {"--gpu-architecture=sm_100a", "--std=c++17", "-default-device"};
    r = N.compile(prog, 3, opts);
    if (r != NVRTC_SUCCESS) {
        size_t n = 0;
        N.log_size(prog, &n);
        std::string log(n, '\0');
        if (n) N.log(prog, &log[0]);
        N.destroy(&prog);
        return nvrtc_fail(r, "nvrtcCompileProgram", log);
    }
    size_t n = 0;
    r = N.cubin_size(prog, &n);
    std::vector<char> cubin(n);
    if (r == NVRTC_SUCCESS) r = N.cubin(prog, cubin.data());
    N.destroy(&prog);
    if (r != NVRTC_SUCCESS) return nvrtc_fail(r, "nvrtcGetCUBIN");
    int rc = cuda_check(cudaLibraryLoadData(&out->lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0),
                        "program compile: cudaLibraryLoadData");
    if (rc) return rc;
    return cuda_check(cudaLibraryGetKernel(&out->kern, out->lib, "bo_prog"), "program compile: cudaLibraryGetKernel");
}

}  // namespace

int jit_compile(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, int layout, JitKernel *out) {
    const Shape shape = jit_shape(prog, t, msize, layout);
    if (shape == kNone)
        return fail(BO_EUNSUPPORTED, "program compile: row-wise programs need msize <= 95 or addresses that stay "
                                     "within 64-word windows (>= 8 accesses per window)");
    if (t > kMaxJitInstructions) return fail(BO_EUNSUPPORTED, "program compile: more than 200000 instructions");
    const std::string src = generate(prog, t, msize, nregs, dtype, shape);
    const size_t key = std::hash<std::string>{}(src);
    std::lock_guard<std::mutex> g(g_mu);               // (compiles are rare: one at a time)
    for (auto &e : g_cache[key])
        if (e.first == src) {
            out->kernel = reinterpret_cast<const void *>(e.second.kern);
            return BO_OK;
        }
    Compiled c{};
    if (int rc = compile_source(src, &c)) return rc;
    g_cache[key].emplace_back(src, c);
    out->kernel = reinterpret_cast<const void *>(c.kern);
    return BO_OK;
}

int launch_jit(const JitKernel &k, void *mem, int64_t p, cudaStream_t st) {
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(static_cast<unsigned>((p + kJitThreads - 1) / kJitThreads));
    cfg.blockDim = dim3(kJitThreads);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    long long pp = p;
    int zero = 0;                       // the generated kernels' opaque zero (see op_expr, CONST)
    void *args[] = {&mem, &pp, &zero};
    cudaLaunchKernelExC(&cfg, k.kernel, args);
    return after_launch("bo_prog (compiled program)");
}

std::string jit_source(const int32_t *prog, int64_t t, int64_t msize, int nregs, int dtype, int layout) {
    const Shape shape = jit_shape(prog, t, msize, layout);
    return shape == kNone ? std::string() : generate(prog, t, msize, nregs, dtype, shape);
}

}  // namespace bo
