// up_host.cpp -- the C ABI of libup.so (include/up.h): context, NVRTC
// specialisation + kernel cache (row a2), launches, column codec, combine.
#include <cuda.h>
#include <dlfcn.h>
#include <sys/stat.h>
#include <unistd.h>
#include <cuda_runtime.h>
#include <nvrtc.h>

#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <iterator>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "../../include/up.h"
#include "codegen.h"
#include "expr.h"
#include "hbig.h"
#include "up_embed.inc"   // k_up_dev_src, k_up_kparams_src (generated from up_dev.cuh / up_kparams.h)
#include "up_kparams.h"

using namespace uph;

// ---------------------------------------------------------------- static kernels (kernels.cu)
extern "C" {
cudaError_t upk_launch_from_bin(const uint32_t *mag, int W, const uint8_t *neg, long long n, const uint32_t *bound,
                                int L, uint32_t *out, long long ld, uint32_t *flags, cudaStream_t st);
cudaError_t upk_launch_to_bin(const uint32_t *planes, int L, long long ld, long long n, uint32_t *mag, uint8_t *neg,
                              cudaStream_t st);
cudaError_t upk_launch_combine(const uint32_t *partials, int nranks, int la, uint32_t *out, cudaStream_t st);
cudaError_t upk_launch_combine_scaled(const uint32_t *partials, int nparts, int la, uint32_t *out, int scaled,
                                      const uint32_t *scale, int nsc, cudaStream_t st);
int upk_contract_tc_slots(int La, int Lb);
cudaError_t upk_launch_contract_tc(const uint32_t *A, long long lda, int La, const uint32_t *B, long long ldb, int Lb,
                                   long long n, int sign, unsigned long long *ws, uint32_t *ticket, uint32_t *result,
                                   int LA, int num_sms, cudaStream_t st);
cudaError_t upk_launch_group_combine(const uint32_t *parts, int nranks, long long part_words,
                                     const unsigned long long *counts, int G, int n_aggs, const void *d_descs,
                                     uint32_t *out, unsigned long long *counts_out, cudaStream_t st);
cudaError_t upk_launch_from_compact(const uint8_t *bytes, int Lb, long long n, const uint32_t *bound, int L,
                                   uint32_t *out, long long ld, uint32_t *flags, cudaStream_t st);
cudaError_t upk_launch_to_compact(const uint32_t *planes, int L, long long ld, long long n, uint8_t *bytes, int Lb,
                                 cudaStream_t st);
cudaError_t upk_launch_planes_to_quads(const uint32_t *planes, int L, long long ld, long long n, uint32_t *quads,
                                      long long ldq, cudaStream_t st);
cudaError_t upk_launch_quads_to_planes(const uint32_t *quads, long long ldq, int L, long long n, uint32_t *planes,
                                      long long ld, cudaStream_t st);
cudaError_t upk_launch_contract_tq(const uint32_t *A, long long lda, int La, const uint32_t *B, long long ldb, int Lb,
                                   long long n, int sign, unsigned long long *ws, uint32_t *ticket, uint32_t *result,
                                   int LA, int num_sms, cudaStream_t st);
}

namespace {

thread_local std::string g_err;

// Driver API entry points fetched through the runtime, so libup.so has no
// link-time dependency on libcuda.so.1 (it loads on GPU-less build hosts).
struct Drv {
    CUresult (*ModuleLoadData)(CUmodule *, const void *) = nullptr;
    CUresult (*ModuleGetFunction)(CUfunction *, CUmodule, const char *) = nullptr;
    CUresult (*ModuleUnload)(CUmodule) = nullptr;
    CUresult (*LaunchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                             CUstream, void **, void **) = nullptr;
    CUresult (*OccupancyMaxActiveBlocksPerMultiprocessor)(int *, CUfunction, int, size_t) = nullptr;
    CUresult (*GetErrorString)(CUresult, const char **) = nullptr;
    CUresult (*FuncSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
    CUresult (*LaunchKernelEx)(const CUlaunchConfig *, CUfunction, void **, void **) = nullptr;
    bool ok = false;
} drv;

cudaError_t load_drv() {
    if (drv.ok) return cudaSuccess;
    cudaDriverEntryPointQueryResult q;
#define UP_ENTRY(name, field)                                                                            \
    do {                                                                                                 \
        cudaError_t e = cudaGetDriverEntryPoint(name, (void **)&drv.field, cudaEnableDefault, &q);      \
        if (e != cudaSuccess) return e;                                                                  \
        if (q != cudaDriverEntryPointSuccess || !drv.field) return cudaErrorSymbolNotFound;              \
    } while (0)
    UP_ENTRY("cuModuleLoadData", ModuleLoadData);
    UP_ENTRY("cuModuleGetFunction", ModuleGetFunction);
    UP_ENTRY("cuModuleUnload", ModuleUnload);
    UP_ENTRY("cuLaunchKernel", LaunchKernel);
    UP_ENTRY("cuOccupancyMaxActiveBlocksPerMultiprocessor", OccupancyMaxActiveBlocksPerMultiprocessor);
    UP_ENTRY("cuGetErrorString", GetErrorString);
    UP_ENTRY("cuFuncSetAttribute", FuncSetAttribute);
    UP_ENTRY("cuLaunchKernelEx", LaunchKernelEx);
#undef UP_ENTRY
    drv.ok = true;
    return cudaSuccess;
}

up_status fail(up_status st, const char *fmt, ...) {
    char buf[2048];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return st;
}

#define CUDA_TRY(x)                                                                          \
    do {                                                                                     \
        cudaError_t e_ = (x);                                                                \
        if (e_ != cudaSuccess) return fail(UP_E_CUDA, "%s: %s", #x, cudaGetErrorString(e_)); \
    } while (0)
#define CU_TRY(x)                                                                         \
    do {                                                                                  \
        CUresult e_ = (x);                                                                \
        if (e_ != CUDA_SUCCESS) {                                                         \
            const char *s_ = nullptr;                                                     \
            if (drv.GetErrorString) drv.GetErrorString(e_, &s_);                          \
            return fail(UP_E_CUDA, "%s: %s", #x, s_ ? s_ : "?");                          \
        }                                                                                 \
    } while (0)

constexpr int kThreads = 256;
constexpr int kWsSlots = 1 << 16;
constexpr int kIngestChunks = 8;          // host ingestion: copy / convert pipeline depth
constexpr size_t kIngestChunkMin = 16u << 20;   // bytes per chunk at least
constexpr int kContractMinProducts = 100;   // row contraction only for compute-bound products
constexpr long kSplitAutoProducts = 80 * 80;  // automatic split from this product size on
constexpr int kWideMinLimbs = 257;  // warp-per-row only beyond this (per-thread measured faster at p <= 1000)

struct JitKernel {
    CUmodule mod = nullptr;
    CUfunction fn = nullptr;
    int rows_per_thread = 1;
    int ws_slots = 0;
    int blocks_per_sm = 1;
    int threads = kThreads;
    int dyn_smem = 0;      // dynamic shared memory per block (bytes)
    int rows_per_block = 0;  // > 0: warp-per-row kernels (rows per block-iteration)
    bool pdl = false;        // may be launched with programmatic stream serialization
    std::string src;
};

}  // namespace

// a split SELECT SUM: top-level column products (tensor-core or CUDA-core
// contraction kernels) + the rest (fused per-thread kernel) + exact combine
struct SplitPlan {
    bool split = false;
    int LAs = 0;
    std::vector<uph::SplitTerm> prods;
    std::vector<JitKernel *> cc_kernels;   // per product: CUDA-core kernel, nullptr = tensor cores
    JitKernel *rest_kernel = nullptr;
    int rest_scale = 0;                    // rest partial x 10^rest_scale in the combine
};

struct up_ctx {
    int device = 0;
    int num_sms = 148;
    unsigned long long *d_ws = nullptr;   // SUM slots
    uint32_t *d_ticket = nullptr;
    uint32_t *d_flags = nullptr;
    void *d_stage = nullptr;
    size_t stage_bytes = 0;
    void *d_scratch = nullptr;   // kernel scratch (sin_P running sums), grown on demand
    size_t scratch_bytes = 0;
    uint32_t *d_parts = nullptr; // per-term SUM partials of a split SUM
    size_t parts_words = 0;
    std::map<int, uint32_t *> pow10_dev;  // 10^p magnitude in up_limbs(p) limbs
    std::unordered_map<std::string, std::unique_ptr<JitKernel>> by_src;
    std::unordered_map<std::string, JitKernel *> by_key;
    std::unordered_map<std::string, SplitPlan> plans;   // split SUM plans (up_sum_expr)
    uint64_t launches = 0;
    double jit_ms = 0.0;
    bool pipelined = false;   // up_set_pipelined: PDL launches of the fused SUM kernels
    // host ingestion: a copy stream and per-chunk events, so the H2D copy of
    // chunk k+1 overlaps the conversion / range check of chunk k
    cudaStream_t copy_st = nullptr;
    cudaEvent_t chunk_ev[kIngestChunks] = {};
    // split SUMs over quad columns: the tensor-core contraction on a side stream
    // (own workspace + ticket) beside the rest kernel on the caller's stream
    cudaStream_t side = nullptr, side_rest = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_join_rest = nullptr;
    unsigned long long *d_ws2 = nullptr;
    uint32_t *d_ticket2 = nullptr;
    std::mutex mu;
};

namespace {

up_status ensure_stage(up_ctx *c, size_t bytes, cudaStream_t st) {
    if (bytes <= c->stage_bytes) return UP_OK;
    if (c->d_stage) {
        CUDA_TRY(cudaStreamSynchronize(st));
        CUDA_TRY(cudaFree(c->d_stage));
        c->d_stage = nullptr;
    }
    size_t nb = std::max(bytes, c->stage_bytes * 2);
    CUDA_TRY(cudaMalloc(&c->d_stage, nb));
    c->stage_bytes = nb;
    return UP_OK;
}

up_status pow10_device(up_ctx *c, int p, const uint32_t **out) {
    auto it = c->pow10_dev.find(p);
    if (it != c->pow10_dev.end()) { *out = it->second; return UP_OK; }
    const int L = limbs_for_precision(p);
    std::vector<uint32_t> w = HBig::pow10(p).twos(L, false);
    uint32_t *d = nullptr;
    CUDA_TRY(cudaMalloc(&d, sizeof(uint32_t) * (size_t)L));
    CUDA_TRY(cudaMemcpy(d, w.data(), sizeof(uint32_t) * (size_t)L, cudaMemcpyHostToDevice));
    c->pow10_dev[p] = d;
    *out = d;
    return UP_OK;
}

up_status check_column(const up_column *col, const char *what) {
    if (!col) return fail(UP_E_INVAL, "%s: null column", what);
    if (col->p < 1 || col->s < 0) return fail(UP_E_INVAL, "%s: bad DECIMAL(%d,%d)", what, col->p, col->s);
    if (col->limbs != limbs_for_precision(col->p))
        return fail(UP_E_INVAL, "%s: limbs %d != up_limbs(%d) = %d", what, col->limbs, col->p, limbs_for_precision(col->p));
    if (col->layout != UP_LAYOUT_PLANES && col->layout != UP_LAYOUT_COMPACT && col->layout != UP_LAYOUT_QUADS)
        return fail(UP_E_INVAL, "%s: unknown layout %d", what, col->layout);
    if (col->layout == UP_LAYOUT_COMPACT) {
        if (col->ld != up_compact_bytes(col->p))
            return fail(UP_E_INVAL, "%s: compact column needs ld = up_compact_bytes(%d) = %d", what, col->p, up_compact_bytes(col->p));
        if (col->n < 0) return fail(UP_E_INVAL, "%s: bad n", what);
        if (col->n > 0 && (!col->data || ((uintptr_t)col->data & 15))) return fail(UP_E_INVAL, "%s: data must be 16-byte aligned device memory", what);
        if (col->n >= (1ll << 32)) return fail(UP_E_UNSUPPORTED, "%s: more than 2^32-1 rows per call", what);
        return UP_OK;
    }
    if (col->n < 0 || col->ld < col->n || (col->ld & 3)) return fail(UP_E_INVAL, "%s: bad n/ld (%lld/%lld)", what, (long long)col->n, (long long)col->ld);
    if (col->n > 0 && (!col->data || ((uintptr_t)col->data & 15))) return fail(UP_E_INVAL, "%s: data must be 16-byte aligned device memory", what);
    if (col->n >= (1ll << 32)) return fail(UP_E_UNSUPPORTED, "%s: more than 2^32-1 rows per call", what);
    return UP_OK;
}

up_status need_planes(const up_column *col, const char *what) {
    if (col && col->layout != UP_LAYOUT_PLANES)
        return fail(UP_E_UNSUPPORTED, "%s: this call needs a limb-plane column (compact and quad columns: up_eval_expr / "
                                      "up_sum_expr / up_filter)", what);
    return UP_OK;
}

const char *kNvrtcOpts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-default-device", "-lineinfo", "-DNDEBUG", "--device-int128"};

// On-disk cubin cache (keyed by FNV-1a of source + options + embedded header):
// $UP_JIT_CACHE, else <dir of libup.so>/_jitcache.  Purely a compile-time
// saving; a miss recompiles with NVRTC.
uint64_t fnv1a(const std::string &s, uint64_t h = 1469598103934665603ull) {
    for (unsigned char ch : s) { h ^= ch; h *= 1099511628211ull; }
    return h;
}
std::string cache_dir() {
    if (const char *e = getenv("UP_JIT_CACHE")) return e;
    Dl_info info;
    if (dladdr((void *)&fnv1a, &info) && info.dli_fname) {
        std::string f = info.dli_fname;
        size_t k = f.rfind('/');
        if (k != std::string::npos) return f.substr(0, k) + "/_jitcache";
    }
    return "";
}
std::string cache_path(const std::string &src) {
    std::string d = cache_dir();
    if (d.empty()) return "";
    uint64_t h = fnv1a(src);
    for (const char *o : kNvrtcOpts) h = fnv1a(o, h);
    h = fnv1a(k_up_dev_src, h);
    h = fnv1a(k_up_kparams_src, h);
    h = fnv1a(k_up_wide_src, h);
    char name[64];
    snprintf(name, sizeof name, "/%016llx.cubin", (unsigned long long)h);
    return d + name;
}
bool read_file(const std::string &path, std::vector<char> &out) {
    std::ifstream f(path, std::ios::binary);
    if (!f) return false;
    out.assign(std::istreambuf_iterator<char>(f), std::istreambuf_iterator<char>());
    return !out.empty();
}
void write_file_atomic(const std::string &path, const std::vector<char> &data) {
    size_t k = path.rfind('/');
    if (k != std::string::npos) mkdir(path.substr(0, k).c_str(), 0755);
    std::string tmp = path + ".tmp" + std::to_string((long)getpid());
    {
        std::ofstream f(tmp, std::ios::binary);
        if (!f) return;
        f.write(data.data(), (std::streamsize)data.size());
    }
    rename(tmp.c_str(), path.c_str());
}

up_status nvrtc_to_cubin(const std::string &src, std::vector<char> &cubin) {
    nvrtcProgram prog;
    const char *hdrs[3] = {k_up_dev_src, k_up_kparams_src, k_up_wide_src};
    const char *names[3] = {"up_dev.cuh", "up_kparams.h", "up_wide.cuh"};
    if (nvrtcCreateProgram(&prog, src.c_str(), "upk.cu", 3, hdrs, names) != NVRTC_SUCCESS)
        return fail(UP_E_NVRTC, "nvrtcCreateProgram failed");
    nvrtcResult r = nvrtcCompileProgram(prog, (int)(sizeof kNvrtcOpts / sizeof kNvrtcOpts[0]), kNvrtcOpts);
    if (r != NVRTC_SUCCESS) {
        size_t ls = 0;
        nvrtcGetProgramLogSize(prog, &ls);
        std::string log(ls, '\0');
        nvrtcGetProgramLog(prog, &log[0]);
        nvrtcDestroyProgram(&prog);
        return fail(UP_E_NVRTC, "NVRTC: %s\n%s", nvrtcGetErrorString(r), log.substr(0, 1500).c_str());
    }
    size_t cs = 0;
    nvrtcGetCUBINSize(prog, &cs);
    cubin.resize(cs);
    nvrtcGetCUBIN(prog, cubin.data());
    nvrtcDestroyProgram(&prog);
    return UP_OK;
}

up_status compile(up_ctx *c, const std::string &src, JitKernel **out) {
    auto it = c->by_src.find(src);
    if (it != c->by_src.end()) { *out = it->second.get(); return UP_OK; }
    auto t0 = std::chrono::steady_clock::now();
    if (const char *dump = getenv("UP_DUMP_DIR")) {
        std::string path = std::string(dump) + "/upk_" + std::to_string(c->by_src.size()) + ".cu";
        std::ofstream(path) << src;
    }
    std::vector<char> cubin;
    const std::string cpath = cache_path(src);
    if (cpath.empty() || !read_file(cpath, cubin)) {
        if (up_status st = nvrtc_to_cubin(src, cubin)) return st;
        if (!cpath.empty()) write_file_atomic(cpath, cubin);
    }
    auto k = std::make_unique<JitKernel>();
    CU_TRY(drv.ModuleLoadData(&k->mod, cubin.data()));
    CU_TRY(drv.ModuleGetFunction(&k->fn, k->mod, "upk"));
    int nb = 0;
    CU_TRY(drv.OccupancyMaxActiveBlocksPerMultiprocessor(&nb, k->fn, kThreads, 0));
    k->blocks_per_sm = std::max(1, nb);
    k->src = src;
    c->jit_ms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = k.get();
    c->by_src[src] = std::move(k);
    return UP_OK;
}

struct Typed {
    std::unique_ptr<Node> root;
    std::vector<ColType> types;
};

up_status type_expr(const char *expr, const up_column *cols, int ncols, Typed &t) {
    if (!expr) return fail(UP_E_INVAL, "null expression");
    if (ncols < 0 || ncols > UP_MAX_COLS) return fail(UP_E_UNSUPPORTED, "at most %d columns", UP_MAX_COLS);
    for (int i = 0; i < ncols; ++i) {
        if (cols[i].p < 1 || cols[i].s < 0 || cols[i].limbs != limbs_for_precision(cols[i].p))
            return fail(UP_E_INVAL, "column %d: bad type/limbs", i + 1);
        t.types.push_back({cols[i].p, cols[i].s, cols[i].limbs,
                           cols[i].layout == UP_LAYOUT_COMPACT ? up_compact_bytes(cols[i].p) : 0,
                           cols[i].layout == UP_LAYOUT_QUADS});
    }
    std::string err;
    t.root = parse_expr(expr, ncols, err);
    if (!t.root) return fail(UP_E_INVAL, "expression '%s': %s", expr, err.c_str());
    if (type_tree(t.root.get(), t.types, err)) return fail(UP_E_INVAL, "expression '%s': %s", expr, err.c_str());
    return UP_OK;
}

std::string key_of(const char *tag, const char *expr, const up_column *cols, int ncols, int extra) {
    std::string k = tag;
    k += '|';
    k += expr;
    for (int i = 0; i < ncols; ++i)
        k += "|" + std::to_string(cols[i].p) + "," + std::to_string(cols[i].s) +
             (cols[i].layout == UP_LAYOUT_COMPACT ? "c" : cols[i].layout == UP_LAYOUT_QUADS ? "q" : "");
    k += "|" + std::to_string(extra);
    if (getenv("UP_NO_OPT")) k += "|noopt";
    if (getenv("UP_NO_WIDE")) k += "|nowide";
    if (getenv("UP_SPLIT")) k += "|split";
    return k;
}

up_status launch(up_ctx *c, JitKernel *k, up_kparams &P, long long n, cudaStream_t st, bool allow_pdl = true) {
    long long per_block = k->rows_per_block > 0 ? k->rows_per_block : (long long)k->threads * k->rows_per_thread;
    long long want = (n + per_block - 1) / per_block;
    long long cap = (long long)k->blocks_per_sm * c->num_sms;
    int grid = (int)std::max(1ll, std::min(want, cap));
    void *args[] = {&P};
    if (k->pdl && c->pipelined && allow_pdl) {
        CUlaunchAttribute at[1];
        at[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
        at[0].value.programmaticStreamSerializationAllowed = 1;
        CUlaunchConfig cfg = {};
        cfg.gridDimX = grid; cfg.gridDimY = 1; cfg.gridDimZ = 1;
        cfg.blockDimX = k->threads; cfg.blockDimY = 1; cfg.blockDimZ = 1;
        cfg.sharedMemBytes = (unsigned)k->dyn_smem;
        cfg.hStream = (CUstream)st;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        CU_TRY(drv.LaunchKernelEx(&cfg, k->fn, args, nullptr));
    } else {
        CU_TRY(drv.LaunchKernel(k->fn, grid, 1, 1, k->threads, 1, 1, (unsigned)k->dyn_smem, (CUstream)st, args, nullptr));
    }
    c->launches++;
    return UP_OK;
}

up_status expr_kernel(up_ctx *c, const char *expr, const up_column *cols, int ncols, bool sum, long long n_global,
                      JitKernel **out, int *LA_out, Node **root_out, Typed &t) {
    up_status s = type_expr(expr, cols, ncols, t);
    if (s) return s;
    const int ps = sum_precision(t.root->p, n_global);
    const int LA = sum ? limbs_for_precision(ps) : 0;
    if (LA_out) *LA_out = LA;
    if (root_out) *root_out = t.root.get();
    std::string key = key_of(sum ? "sum" : "eval", expr, cols, ncols, LA);
    auto it = c->by_key.find(key);
    if (it != c->by_key.end()) { *out = it->second; return UP_OK; }
    GenOpts o;
    o.sum = sum;
    o.LA = LA;
    GenInfo info;
    std::string src;
    // expression optimiser (alignment scheduling + constant pre-calculation),
    // value-preserving; the kernel is generated from the optimised tree
    std::unique_ptr<Node> opt_root = getenv("UP_NO_OPT") ? nullptr : optimize(t.root.get(), t.types);
    const Node *gen_root = opt_root ? opt_root.get() : t.root.get();
    // wide SUM regime: warp per row, linear decomposition into summed terms
    bool any_compact = false;
    for (const ColType &ct : t.types) any_compact = any_compact || ct.Lb > 0 || ct.Q;   // wide regime reads planes
    if (sum && !any_compact && max_limbs(gen_root) >= kWideMinLimbs && LA <= 512 && !getenv("UP_NO_WIDE"))
        src = gen_wide_sum_kernel(gen_root, t.types, LA, info);
    if (src.empty()) {
        info = GenInfo();
        src = gen_expr_kernel(gen_root, t.types, o, info);
    }
    if (sum && info.ws_slots > kWsSlots) return fail(UP_E_UNSUPPORTED, "SUM too wide (%d slots)", info.ws_slots);
    JitKernel *k = nullptr;
    s = compile(c, src, &k);
    if (s) return s;
    k->rows_per_thread = info.rows_per_thread;
    k->ws_slots = info.ws_slots;
    k->rows_per_block = info.rows_per_block;
    k->pdl = info.pdl;
    if (info.threads != k->threads || info.dyn_smem != k->dyn_smem) {
        k->threads = info.threads;
        if (info.dyn_smem > 0)
            CU_TRY(drv.FuncSetAttribute(k->fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, info.dyn_smem));
        k->dyn_smem = info.dyn_smem;
        int nb = 0;
        CU_TRY(drv.OccupancyMaxActiveBlocksPerMultiprocessor(&nb, k->fn, k->threads, (size_t)k->dyn_smem));
        k->blocks_per_sm = std::max(1, nb);
    }
    c->by_key[key] = k;
    *out = k;
    return UP_OK;
}

// compile (or fetch) a kernel generated by `gen` under `key`, applying its launch info
template <class Gen>
up_status kernel_for(up_ctx *c, const std::string &key, Gen gen, JitKernel **out) {
    auto it = c->by_key.find(key);
    if (it != c->by_key.end()) { *out = it->second; return UP_OK; }
    GenInfo info;
    std::string src = gen(info);
    if (src.empty()) return fail(UP_E_UNSUPPORTED, "no kernel for %s", key.c_str());
    if (info.ws_slots > kWsSlots) return fail(UP_E_UNSUPPORTED, "SUM too wide (%d slots)", info.ws_slots);
    JitKernel *k = nullptr;
    if (up_status s = compile(c, src, &k)) return s;
    k->rows_per_thread = info.rows_per_thread;
    k->ws_slots = info.ws_slots;
    k->rows_per_block = info.rows_per_block;
    if (info.threads != k->threads || info.dyn_smem != k->dyn_smem) {
        k->threads = info.threads;
        if (info.dyn_smem > 0)
            CU_TRY(drv.FuncSetAttribute(k->fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, info.dyn_smem));
        k->dyn_smem = info.dyn_smem;
        int nb = 0;
        CU_TRY(drv.OccupancyMaxActiveBlocksPerMultiprocessor(&nb, k->fn, k->threads, (size_t)k->dyn_smem));
        k->blocks_per_sm = std::max(1, nb);
    }
    c->by_key[key] = k;
    *out = k;
    return UP_OK;
}

void fill_cols(up_kparams &P, const up_column *cols, int ncols) {
    memset(&P, 0, sizeof P);
    for (int i = 0; i < ncols; ++i) {
        P.col[i] = cols[i].data;
        P.ld[i] = cols[i].ld;
    }
    P.n = ncols ? cols[0].n : 0;
}

}  // namespace

up_status scratch_locked(up_ctx *c, size_t bytes, void **out);   // ctx scratch; caller holds c->mu

// ====================================================================== C ABI
extern "C" {

const char *up_last_error(void) { return g_err.c_str(); }

int32_t up_limbs(int32_t p) { return limbs_for_precision(p); }
int32_t up_quads(int32_t p) { return (limbs_for_precision(p) + 1 + 3) / 4; }
int64_t up_ld(int64_t n) { return (n + 3) & ~3ll; }
int32_t up_sum_precision(int32_t p, int64_t n_global) { return sum_precision(p, n_global); }

up_status up_ctx_create(int device, up_ctx **out) {
    if (!out) return fail(UP_E_INVAL, "null out");
    CUDA_TRY(cudaSetDevice(device));
    CUDA_TRY(cudaFree(nullptr));   // initialise the primary context (shared with torch)
    CUDA_TRY(load_drv());
    auto c = std::make_unique<up_ctx>();
    c->device = device;
    CUDA_TRY(cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device));
    CUDA_TRY(cudaMalloc(&c->d_ws, sizeof(unsigned long long) * kWsSlots));
    CUDA_TRY(cudaMemset(c->d_ws, 0, sizeof(unsigned long long) * kWsSlots));
    CUDA_TRY(cudaMalloc(&c->d_ticket, 64));
    CUDA_TRY(cudaMemset(c->d_ticket, 0, 64));
    CUDA_TRY(cudaMalloc(&c->d_flags, 64));
    CUDA_TRY(cudaMemset(c->d_flags, 0, 64));
    CUDA_TRY(cudaDeviceSynchronize());
    *out = c.release();
    return UP_OK;
}

up_status up_set_pipelined(up_ctx *c, int on) {
    if (!c) return fail(UP_E_INVAL, "null ctx");
    c->pipelined = on != 0;
    return UP_OK;
}

up_status up_ctx_destroy(up_ctx *c) {
    if (!c) return UP_OK;
    cudaDeviceSynchronize();
    for (auto &kv : c->by_src) if (kv.second->mod && drv.ModuleUnload) drv.ModuleUnload(kv.second->mod);
    for (auto &kv : c->pow10_dev) cudaFree(kv.second);
    cudaFree(c->d_ws);
    cudaFree(c->d_ticket);
    cudaFree(c->d_flags);
    if (c->d_stage) cudaFree(c->d_stage);
    for (cudaEvent_t e : c->chunk_ev) if (e) cudaEventDestroy(e);
    if (c->copy_st) cudaStreamDestroy(c->copy_st);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->ev_join_rest) cudaEventDestroy(c->ev_join_rest);
    if (c->side) cudaStreamDestroy(c->side);
    if (c->side_rest) cudaStreamDestroy(c->side_rest);
    if (c->d_ws2) cudaFree(c->d_ws2);
    if (c->d_ticket2) cudaFree(c->d_ticket2);
    if (c->d_scratch) cudaFree(c->d_scratch);
    if (c->d_parts) cudaFree(c->d_parts);
    delete c;
    return UP_OK;
}

uint64_t up_launch_count(up_ctx *c) { return c ? c->launches : 0; }
double up_jit_ms(up_ctx *c) { return c ? c->jit_ms : 0.0; }

up_status up_column_from_device_bin(up_ctx *c, const uint32_t *d_mag, int32_t W, const uint8_t *d_neg,
                                    up_column *dst, void *stream) {
    if (!c) return fail(UP_E_INVAL, "null ctx");
    if (up_status s = check_column(dst, "dst")) return s;
    if (W < 1) return fail(UP_E_INVAL, "mag_words must be >= 1");
    if (dst->n == 0) return UP_OK;
    std::lock_guard<std::mutex> g(c->mu);
    const uint32_t *bound = nullptr;
    if (up_status s = pow10_device(c, dst->p, &bound)) return s;
    if (dst->layout == UP_LAYOUT_COMPACT) {   // via limb planes in the ctx scratch
        const long long ld = (dst->n + 3) & ~3ll;
        uint32_t *planes = nullptr;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)dst->limbs * (size_t)ld, (void **)&planes)) return s;
        CUDA_TRY(upk_launch_from_bin(d_mag, W, d_neg, dst->n, bound, dst->limbs, planes, ld, c->d_flags, (cudaStream_t)stream));
        CUDA_TRY(upk_launch_to_compact(planes, dst->limbs, ld, dst->n, (uint8_t *)dst->data, (int)dst->ld, (cudaStream_t)stream));
        c->launches += 2;
        return UP_OK;
    }
    if (dst->layout == UP_LAYOUT_QUADS) {   // via limb planes in the ctx scratch
        const long long ld = (dst->n + 3) & ~3ll;
        uint32_t *planes = nullptr;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)dst->limbs * (size_t)ld, (void **)&planes)) return s;
        CUDA_TRY(upk_launch_from_bin(d_mag, W, d_neg, dst->n, bound, dst->limbs, planes, ld, c->d_flags, (cudaStream_t)stream));
        CUDA_TRY(upk_launch_planes_to_quads(planes, dst->limbs, ld, dst->n, dst->data, dst->ld, (cudaStream_t)stream));
        c->launches += 2;
        return UP_OK;
    }
    CUDA_TRY(upk_launch_from_bin(d_mag, W, d_neg, dst->n, bound, dst->limbs, dst->data, dst->ld, c->d_flags,
                                 (cudaStream_t)stream));
    c->launches++;
    return UP_OK;
}

up_status up_column_from_host_bin(up_ctx *c, const uint32_t *mag, int32_t W, const uint8_t *neg, up_column *dst,
                                  void *stream) {
    if (!c) return fail(UP_E_INVAL, "null ctx");
    if (up_status s = check_column(dst, "dst")) return s;
    if (W < 1) return fail(UP_E_INVAL, "mag_words must be >= 1");
    if (dst->n == 0) return UP_OK;
    cudaStream_t st = (cudaStream_t)stream;
    const size_t mb = sizeof(uint32_t) * (size_t)W * (size_t)dst->n, nb = neg ? (size_t)dst->n : 0;
    const size_t mb_al = (mb + 255) & ~(size_t)255;
    {
        std::lock_guard<std::mutex> g(c->mu);
        if (up_status s = ensure_stage(c, mb_al + nb, st)) return s;
        CUDA_TRY(cudaMemcpyAsync(c->d_stage, mag, mb, cudaMemcpyHostToDevice, st));
        if (neg) CUDA_TRY(cudaMemcpyAsync((char *)c->d_stage + mb_al, neg, nb, cudaMemcpyHostToDevice, st));
    }
    if (up_status s = up_column_from_device_bin(c, (const uint32_t *)c->d_stage, W,
                                                neg ? (const uint8_t *)((char *)c->d_stage + mb_al) : nullptr, dst,
                                                stream))
        return s;
    // up.h: the caller may reuse or free the host buffers when this returns
    CUDA_TRY(cudaStreamSynchronize(st));
    return UP_OK;
}

up_status up_column_from_host(up_ctx *c, const char *const *decimals, up_column *dst, void *stream) {
    if (!c || !decimals) return fail(UP_E_INVAL, "null argument");
    if (up_status s = check_column(dst, "dst")) return s;
    const long long n = dst->n;
    const int L = dst->limbs;
    std::vector<uint32_t> mag((size_t)n * (size_t)L, 0);
    std::vector<uint8_t> neg((size_t)n, 0);
    const HBig bound = HBig::pow10(dst->p);
    for (long long i = 0; i < n; ++i) {
        const char *p = decimals[i];
        if (!p) return fail(UP_E_INVAL, "row %lld: null string", i);
        while (*p == ' ') ++p;
        bool ng = false;
        if (*p == '-' || *p == '+') { ng = (*p == '-'); ++p; }
        std::string ip, fp;
        while (*p >= '0' && *p <= '9') ip += *p++;
        if (*p == '.') { ++p; while (*p >= '0' && *p <= '9') fp += *p++; }
        while (*p == ' ') ++p;
        if (*p || (ip.empty() && fp.empty())) return fail(UP_E_INVAL, "row %lld: bad decimal '%s'", i, decimals[i]);
        if ((int)fp.size() > dst->s) return fail(UP_E_RANGE, "row %lld: more than %d fraction digits", i, dst->s);
        fp.append((size_t)(dst->s - (int)fp.size()), '0');
        HBig m;
        HBig::from_dec(ip + fp, m);
        if (HBig::cmp(m, bound) >= 0) return fail(UP_E_RANGE, "row %lld: '%s' exceeds DECIMAL(%d,%d)", i, decimals[i], dst->p, dst->s);
        for (int j = 0; j < L; ++j) mag[(size_t)i * L + j] = m.limb((size_t)j);
        neg[(size_t)i] = (ng && !m.is_zero()) ? 1 : 0;
    }
    up_status s = up_column_from_host_bin(c, mag.data(), L, neg.data(), dst, stream);
    if (s) return s;
    CUDA_TRY(cudaStreamSynchronize((cudaStream_t)stream));   // host temporaries die here
    return UP_OK;
}

int32_t up_compact_bytes(int32_t p) {
    // Lb = ceil((1 + p log2 10) / 8), exactly: bitlen(10^p - 1) + 1 sign bit, in bytes
    if (p < 1) return 1;
    HBig m = HBig::sub(HBig::pow10(p), HBig(1));
    return (m.bitlen() + 1 + 7) / 8;
}

up_status up_column_from_device_compact(up_ctx *c, const uint8_t *d_bytes, up_column *dst, void *stream) {
    if (!c) return fail(UP_E_INVAL, "null ctx");
    if (up_status s = check_column(dst, "dst")) return s;
    if (dst->n == 0) return UP_OK;
    std::lock_guard<std::mutex> g(c->mu);
    const uint32_t *bound = nullptr;
    if (up_status s = pow10_device(c, dst->p, &bound)) return s;
    if (dst->layout == UP_LAYOUT_COMPACT) {   // stays compact: copy + range check (no planes written)
        const size_t nb = (size_t)dst->ld * (size_t)dst->n;
        if ((const void *)d_bytes != (const void *)dst->data)
            CUDA_TRY(cudaMemcpyAsync(dst->data, d_bytes, nb, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
        CUDA_TRY(upk_launch_from_compact((const uint8_t *)dst->data, (int)dst->ld, dst->n, bound, dst->limbs, nullptr, 0,
                                         c->d_flags, (cudaStream_t)stream));
        c->launches++;
        return UP_OK;
    }
    if (dst->layout == UP_LAYOUT_QUADS) {   // via limb planes in the ctx scratch
        const long long ld = (dst->n + 3) & ~3ll;
        uint32_t *planes = nullptr;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)dst->limbs * (size_t)ld, (void **)&planes)) return s;
        CUDA_TRY(upk_launch_from_compact(d_bytes, up_compact_bytes(dst->p), dst->n, bound, dst->limbs, planes, ld,
                                         c->d_flags, (cudaStream_t)stream));
        CUDA_TRY(upk_launch_planes_to_quads(planes, dst->limbs, ld, dst->n, dst->data, dst->ld, (cudaStream_t)stream));
        c->launches += 2;
        return UP_OK;
    }
    CUDA_TRY(upk_launch_from_compact(d_bytes, up_compact_bytes(dst->p), dst->n, bound, dst->limbs, dst->data, dst->ld,
                                     c->d_flags, (cudaStream_t)stream));
    c->launches++;
    return UP_OK;
}

// Host compact rows -> dst in chunks of rows: the copy of chunk k+1 (ctx copy
// stream) overlaps the conversion or range check of chunk k (the caller's
// stream, after the chunk's event), so only the last chunk's kernel is
// exposed behind the host link.
up_status up_column_from_host_compact(up_ctx *c, const uint8_t *bytes, up_column *dst, void *stream) {
    if (!c || !bytes) return fail(UP_E_INVAL, "null argument");
    if (up_status s = check_column(dst, "dst")) return s;
    if (dst->n == 0) return UP_OK;
    cudaStream_t st = (cudaStream_t)stream;
    const int Lb = up_compact_bytes(dst->p);
    const long long n = dst->n;
    const size_t nb = (size_t)Lb * (size_t)n;
    std::lock_guard<std::mutex> g(c->mu);
    if (!c->copy_st) {
        CUDA_TRY(cudaStreamCreateWithFlags(&c->copy_st, cudaStreamNonBlocking));
        for (cudaEvent_t &e : c->chunk_ev) CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    const uint32_t *bound = nullptr;
    if (up_status s = pow10_device(c, dst->p, &bound)) return s;
    // destination of the raw rows: in place (compact column) or the ctx stage
    uint8_t *raw = nullptr;
    if (dst->layout == UP_LAYOUT_COMPACT) raw = (uint8_t *)dst->data;
    else {
        if (up_status s = ensure_stage(c, nb, st)) return s;
        raw = (uint8_t *)c->d_stage;
    }
    uint32_t *planes = dst->data;
    long long ld = dst->ld;
    if (dst->layout == UP_LAYOUT_QUADS) {   // via limb planes in the ctx scratch
        ld = (n + 3) & ~3ll;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)dst->limbs * (size_t)ld, (void **)&planes)) return s;
    }
    const int nck = (int)std::max<size_t>(1, std::min<size_t>(kIngestChunks, nb / kIngestChunkMin));
    // rows landing in place (compact column): the copies wait for the caller's
    // prior work on `stream`, which may still read the column.  Into the ctx
    // stage they need not: every call that uses the stage synchronises before
    // returning, so the copies may overlap kernels still queued on `stream`
    // (e.g. the SUM over the previous chunk of a streamed input)
    if (dst->layout == UP_LAYOUT_COMPACT) {
        CUDA_TRY(cudaEventRecord(c->chunk_ev[0], st));
        CUDA_TRY(cudaStreamWaitEvent(c->copy_st, c->chunk_ev[0], 0));
    }
    for (int k = 0; k < nck; ++k) {
        // chunk boundaries on 256-row multiples: 4-byte-aligned compact rows for the kernel's word loads
        const long long r0 = (n * k / nck) & ~255ll, r1 = k + 1 == nck ? n : (n * (k + 1) / nck) & ~255ll;
        if (r1 == r0) continue;
        CUDA_TRY(cudaMemcpyAsync(raw + (size_t)r0 * Lb, bytes + (size_t)r0 * Lb, (size_t)(r1 - r0) * Lb,
                                 cudaMemcpyHostToDevice, c->copy_st));
        CUDA_TRY(cudaEventRecord(c->chunk_ev[k], c->copy_st));
        CUDA_TRY(cudaStreamWaitEvent(st, c->chunk_ev[k], 0));
        if (dst->layout == UP_LAYOUT_COMPACT) {   // rows landed in place: range check only
            CUDA_TRY(upk_launch_from_compact(raw + (size_t)r0 * Lb, Lb, r1 - r0, bound, dst->limbs, nullptr, 0, c->d_flags, st));
        } else {
            CUDA_TRY(upk_launch_from_compact(raw + (size_t)r0 * Lb, Lb, r1 - r0, bound, dst->limbs, planes + r0, ld,
                                             c->d_flags, st));
            if (dst->layout == UP_LAYOUT_QUADS) {
                CUDA_TRY(upk_launch_planes_to_quads(planes + r0, dst->limbs, ld, r1 - r0, dst->data + 4 * r0, dst->ld, st));
                c->launches++;
            }
        }
        c->launches++;
    }
    CUDA_TRY(cudaStreamSynchronize(st));   // up.h: host buffer reusable on return
    return UP_OK;
}

up_status up_column_to_host_compact(up_ctx *c, const up_column *col, uint8_t *bytes, void *stream) {
    if (!c || !bytes) return fail(UP_E_INVAL, "null argument");
    if (up_status s = check_column(col, "col")) return s;
    if (col->n == 0) return UP_OK;
    cudaStream_t st = (cudaStream_t)stream;
    const int Lb = up_compact_bytes(col->p);
    const size_t nb = (size_t)Lb * (size_t)col->n;
    if (col->layout == UP_LAYOUT_COMPACT) {
        CUDA_TRY(cudaMemcpyAsync(bytes, col->data, nb, cudaMemcpyDeviceToHost, st));
        CUDA_TRY(cudaStreamSynchronize(st));
        return UP_OK;
    }
    std::lock_guard<std::mutex> g(c->mu);
    if (up_status s = ensure_stage(c, nb, st)) return s;
    const uint32_t *planes = col->data;
    long long ld = col->ld;
    if (col->layout == UP_LAYOUT_QUADS) {   // quads -> limb planes in the ctx scratch first
        ld = (col->n + 3) & ~3ll;
        uint32_t *pl = nullptr;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)col->limbs * (size_t)ld, (void **)&pl)) return s;
        CUDA_TRY(upk_launch_quads_to_planes(col->data, col->ld, col->limbs, col->n, pl, ld, st));
        c->launches++;
        planes = pl;
    }
    CUDA_TRY(upk_launch_to_compact(planes, col->limbs, ld, col->n, (uint8_t *)c->d_stage, Lb, st));
    c->launches++;
    CUDA_TRY(cudaMemcpyAsync(bytes, c->d_stage, nb, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    return UP_OK;
}

up_status up_column_to_host_bin(up_ctx *c, const up_column *col, uint32_t *mag, uint8_t *neg, void *stream) {
    if (!c || !mag || !neg) return fail(UP_E_INVAL, "null argument");
    if (up_status s = check_column(col, "col")) return s;
    if (col->n == 0) return UP_OK;
    cudaStream_t st = (cudaStream_t)stream;
    const size_t mb = sizeof(uint32_t) * (size_t)col->limbs * (size_t)col->n, nb = (size_t)col->n;
    const size_t mb_al = (mb + 255) & ~(size_t)255;
    std::lock_guard<std::mutex> g(c->mu);
    if (up_status s = ensure_stage(c, mb_al + nb, st)) return s;
    uint32_t *dm = (uint32_t *)c->d_stage;
    uint8_t *dn = (uint8_t *)c->d_stage + mb_al;
    const uint32_t *planes = col->data;
    long long ld = col->ld;
    if (col->layout == UP_LAYOUT_COMPACT) {   // compact -> limb planes in the ctx scratch first
        ld = (col->n + 3) & ~3ll;
        uint32_t *pl = nullptr;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)col->limbs * (size_t)ld, (void **)&pl)) return s;
        const uint32_t *bound = nullptr;
        if (up_status s = pow10_device(c, col->p, &bound)) return s;
        CUDA_TRY(upk_launch_from_compact((const uint8_t *)col->data, (int)col->ld, col->n, bound, col->limbs, pl, ld,
                                         c->d_flags, st));
        c->launches++;
        planes = pl;
    } else if (col->layout == UP_LAYOUT_QUADS) {   // quads -> limb planes in the ctx scratch first
        ld = (col->n + 3) & ~3ll;
        uint32_t *pl = nullptr;
        if (up_status s = scratch_locked(c, sizeof(uint32_t) * (size_t)col->limbs * (size_t)ld, (void **)&pl)) return s;
        CUDA_TRY(upk_launch_quads_to_planes(col->data, col->ld, col->limbs, col->n, pl, ld, st));
        c->launches++;
        planes = pl;
    }
    CUDA_TRY(upk_launch_to_bin(planes, col->limbs, ld, col->n, dm, dn, st));
    c->launches++;
    CUDA_TRY(cudaMemcpyAsync(mag, dm, mb, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaMemcpyAsync(neg, dn, nb, cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    return UP_OK;
}

up_status up_expr_type(up_ctx *c, const char *expr, const up_column *cols, int ncols, int32_t *p, int32_t *s) {
    (void)c;
    Typed t;
    if (up_status st = type_expr(expr, cols, ncols, t)) return st;
    if (p) *p = t.root->p;
    if (s) *s = t.root->s;
    return UP_OK;
}

up_status up_sum_type(up_ctx *c, const char *expr, const up_column *cols, int ncols, int64_t n_global, int32_t *p,
                      int32_t *s, int32_t *la) {
    (void)c;
    Typed t;
    if (up_status st = type_expr(expr, cols, ncols, t)) return st;
    const long long N = n_global > 0 ? n_global : (ncols ? cols[0].n : 0);
    const int ps = sum_precision(t.root->p, N);
    if (p) *p = ps;
    if (s) *s = t.root->s;
    if (la) *la = limbs_for_precision(ps);
    return UP_OK;
}

up_status up_eval_expr(up_ctx *c, const char *expr, const up_column *cols, int ncols, up_column *out, void *stream) {
    if (!c || !cols || ncols < 1) return fail(UP_E_INVAL, "need a ctx and at least one column");
    for (int i = 0; i < ncols; ++i) {
        if (up_status s = check_column(&cols[i], "input")) return s;
        if (cols[i].n != cols[0].n) return fail(UP_E_INVAL, "columns differ in length");
    }
    if (up_status s = check_column(out, "out")) return s;
    if (out->layout != UP_LAYOUT_PLANES) return fail(UP_E_UNSUPPORTED, "out must be limb planes");
    std::lock_guard<std::mutex> g(c->mu);
    JitKernel *k = nullptr;
    Node *root = nullptr;
    Typed t;
    if (up_status s = expr_kernel(c, expr, cols, ncols, false, 0, &k, nullptr, &root, t)) return s;
    if (out->p != root->p || out->s != root->s || out->n != cols[0].n)
        return fail(UP_E_INVAL, "out must be DECIMAL(%d,%d) with %lld rows", root->p, root->s, (long long)cols[0].n);
    up_kparams P;
    fill_cols(P, cols, ncols);
    P.out = out->data;
    P.ld_out = out->ld;
    P.flags = c->d_flags;
    if (P.n == 0) return UP_OK;
    return launch(c, k, P, P.n, (cudaStream_t)stream);
}

up_status up_filter(up_ctx *c, const char *lhs, const char *op, const char *rhs, const up_column *cols, int ncols,
                    int32_t *d_ids, void *stream) {
    if (!c || !cols || ncols < 1 || (!d_ids && cols[0].n > 0) || !lhs || !rhs || !op)
        return fail(UP_E_INVAL, "need a ctx, columns, both sides, an operator and d_ids");
    for (int i = 0; i < ncols; ++i) {
        if (up_status s = check_column(&cols[i], "input")) return s;
        if (cols[i].n != cols[0].n) return fail(UP_E_INVAL, "columns differ in length");
    }
    const std::string o(op);
    int cmp = 0;
    if (o == "<") cmp = CMP_LT;
    else if (o == "<=") cmp = CMP_LE;
    else if (o == ">") cmp = CMP_GT;
    else if (o == ">=") cmp = CMP_GE;
    else if (o == "=" || o == "==") cmp = CMP_EQ;
    else if (o == "<>" || o == "!=") cmp = CMP_NE;
    else return fail(UP_E_INVAL, "unknown comparison operator '%s'", op);
    // the exact difference lhs - rhs, typed by the paper's rules:
    // its sign decides every comparison
    const std::string diff = "(" + std::string(lhs) + ") - (" + std::string(rhs) + ")";
    std::lock_guard<std::mutex> g(c->mu);
    Typed t;
    if (up_status s = type_expr(diff.c_str(), cols, ncols, t)) return s;
    JitKernel *k = nullptr;
    const std::string key = key_of("cmp", diff.c_str(), cols, ncols, cmp);
    auto gen = [&](GenInfo &info) {
        std::unique_ptr<Node> opt_root = getenv("UP_NO_OPT") ? nullptr : optimize(t.root.get(), t.types);
        GenOpts go;
        go.cmp = cmp;
        return gen_expr_kernel(opt_root ? opt_root.get() : t.root.get(), t.types, go, info);
    };
    if (up_status s = kernel_for(c, key, gen, &k)) return s;
    up_kparams P;
    fill_cols(P, cols, ncols);
    P.out = reinterpret_cast<uint32_t *>(d_ids);
    P.flags = c->d_flags;
    if (P.n == 0) return UP_OK;
    return launch(c, k, P, P.n, (cudaStream_t)stream);
}

up_status up_sum_expr(up_ctx *c, const char *expr, const up_column *cols, int ncols, int64_t n_global,
                      uint32_t *d_partial, void *stream) {
    if (!c || !cols || ncols < 1 || !d_partial) return fail(UP_E_INVAL, "need a ctx, columns and d_partial");
    for (int i = 0; i < ncols; ++i) {
        if (up_status s = check_column(&cols[i], "input")) return s;
        if (cols[i].n != cols[0].n) return fail(UP_E_INVAL, "columns differ in length");
    }
    std::lock_guard<std::mutex> g(c->mu);
    JitKernel *k = nullptr;
    int LA = 0;
    Typed t;
    const long long N = n_global > 0 ? n_global : cols[0].n;
    if (N < cols[0].n) return fail(UP_E_INVAL, "n_global < local rows");
    // Split SUM: top-level column products -> row-contraction kernels, the
    // rest -> the fused per-thread kernel, then an exact combine (SUM is
    // linear).  With the tensor-core contraction (contract_tc.cu, default)
    // every top-level column product of >= kContractMinProducts limb products
    // is split off (cfg3 p = 200: 4.4e9 -> 1.1e10 rows/s); the CUDA-core
    // contraction (UP_NO_TC, and beyond 2^31 rows per call) only from
    // kSplitAutoProducts.  Test switches: UP_SPLIT forces, UP_NO_SPLIT disables.
    // (TMA row coordinates are 32-bit signed: more rows per call take the CUDA-core contraction)
    const bool use_tc = getenv("UP_NO_TC") == nullptr && cols[0].n < (1ll << 31);
    bool try_split = getenv("UP_SPLIT") != nullptr;
    bool any_compact = false;
    for (int i = 0; i < ncols; ++i) any_compact = any_compact || cols[i].layout == UP_LAYOUT_COMPACT;
    if (any_compact) try_split = false;   // the row contractions read limb planes (TMA boxes)
    else if (!try_split && !getenv("UP_NO_SPLIT")) {
        const long thr = use_tc ? kContractMinProducts : kSplitAutoProducts;
        for (int i = 0; i < ncols && !try_split; ++i)
            for (int j = 0; j < ncols && !try_split; ++j)
                if ((long)cols[i].limbs * cols[j].limbs >= thr) try_split = true;
    }
    if (try_split && !getenv("UP_NO_SPLIT")) {
        // the split plan (terms, kernels) is cached per (expression, column types, N, knobs):
        // typing, optimising and splitting cost host time on every call otherwise
        // quad contractions address rows as 2 u64 per row in 32-bit TMA coordinates
        const bool quad_tc = use_tc && cols[0].n < (1ll << 30);
        std::string pkey = key_of("splitplan", expr, cols, ncols, 0) + "|" + std::to_string(N) + (use_tc ? "|tc" : "") +
                           (quad_tc ? "|qtc" : "");
        auto pit = c->plans.find(pkey);
        if (pit == c->plans.end()) {
            SplitPlan pl;
            Typed ts;
            if (up_status s = type_expr(expr, cols, ncols, ts)) return s;
            pl.LAs = limbs_for_precision(sum_precision(ts.root->p, N));
            std::unique_ptr<Node> opt_root = getenv("UP_NO_OPT") ? nullptr : optimize(ts.root.get(), ts.types);
            const Node *base = opt_root ? opt_root.get() : ts.root.get();
            std::unique_ptr<Node> rest;
            pl.split = pl.LAs <= 512 && split_sum_terms(base, ts.types, kContractMinProducts, pl.prods, rest, pl.rest_scale);
            if (pl.split) {
                const int LAs = pl.LAs;
                for (const SplitTerm &st : pl.prods) {
                    const int La = cols[st.col_a].limbs, Lb = cols[st.col_b].limbs;
                    JitKernel *kc = nullptr;
                    const bool qa = cols[st.col_a].layout == UP_LAYOUT_QUADS, qb = cols[st.col_b].layout == UP_LAYOUT_QUADS;
                    const bool tc_ok = use_tc && upk_contract_tc_slots(La, Lb) <= kWsSlots;
                    // quad columns: the tensor-core contraction reads both operands as quads;
                    // otherwise the whole SUM stays in the fused kernel
                    if ((qa || qb) && !(qa && qb && tc_ok && quad_tc)) { pl.split = false; break; }
                    if (!tc_ok) {
                        std::string key = "contract|" + std::to_string(La) + "|" + std::to_string(Lb) + "|" + std::to_string(LAs) +
                                          "|" + std::to_string(st.sign) + "|" + std::to_string(st.col_a) + "|" + std::to_string(st.col_b);
                        if (up_status s = kernel_for(c, key, [&](GenInfo &info) {
                                return gen_contract_kernel(La, Lb, LAs, st.sign, st.col_a, st.col_b, info); }, &kc))
                            return s;
                    }
                    pl.cc_kernels.push_back(kc);   // nullptr: tensor-core contraction
                }
                if (pl.split && rest) {
                    std::string key = "rest|" + canonical(rest.get()) + "|" + std::to_string(LAs);
                    for (int i = 0; i < ncols; ++i)
                        key += "|" + std::to_string(cols[i].p) + "," + std::to_string(cols[i].s) + "," + std::to_string(cols[i].layout);
                    Node *rr = rest.get();
                    if (up_status s = kernel_for(c, key, [&](GenInfo &info) {
                            GenOpts o;
                            o.sum = true;
                            o.LA = LAs;
                            return gen_expr_kernel(rr, ts.types, o, info); }, &pl.rest_kernel))
                        return s;
                }
            }
            pit = c->plans.emplace(pkey, std::move(pl)).first;
        }
        const SplitPlan &pl = pit->second;
        if (pl.split) {
            const int LAs = pl.LAs;
            const int T = (int)pl.prods.size() + (pl.rest_kernel ? 1 : 0);
            const size_t need = (size_t)T * (size_t)LAs;
            if (need > c->parts_words) {
                if (c->d_parts) {
                    CUDA_TRY(cudaStreamSynchronize((cudaStream_t)stream));
                    if (c->side) CUDA_TRY(cudaStreamSynchronize(c->side));
                    if (c->side_rest) CUDA_TRY(cudaStreamSynchronize(c->side_rest));
                    CUDA_TRY(cudaFree(c->d_parts));
                }
                CUDA_TRY(cudaMalloc(&c->d_parts, sizeof(uint32_t) * need * 2));
                c->parts_words = need * 2;
            }
            up_kparams P;
            fill_cols(P, cols, ncols);
            P.ws = c->d_ws;
            P.ticket = c->d_ticket;
            P.flags = c->d_flags;
            // quad contractions + a rest kernel: the contraction (6 warps and its
            // shared-memory stages, HBM-bound) and the integer-bound rest kernel
            // run side by side on two ctx streams forked from the caller's stream
            // (the contraction with its own workspace and ticket), joined before
            // the combine.  Both off the caller's stream: on the legacy default
            // stream the pair overlapped less (0.77 vs 0.68 ms, profiles/r02_s66).
            // UP_SERIAL_SPLIT: everything on the caller's stream, back to back.
            // Only for contractions of at most two roles per row block (p <= ~600):
            // with more, the contraction's own MMA / copy overlap is the limit and
            // sharing the SMs slows it more than the division gains (p = 1000:
            // 3.76 vs 3.56 ms back to back, profiles/r02_s67)
            bool overlap = pl.rest_kernel != nullptr && !getenv("UP_SERIAL_SPLIT");
            for (size_t q = 0; q < pl.prods.size() && overlap; ++q) {
                const int ga = (cols[pl.prods[q].col_a].limbs + 4) / 4, gb = (cols[pl.prods[q].col_b].limbs + 4) / 4;
                overlap = !pl.cc_kernels[q] && cols[pl.prods[q].col_a].layout == UP_LAYOUT_QUADS &&
                          ((ga + 7) / 8) * ((gb + 31) / 32) <= 2;
            }
            cudaStream_t tcs = (cudaStream_t)stream;
            unsigned long long *tws = c->d_ws;
            uint32_t *ttk = c->d_ticket;
            if (overlap) {
                if (!c->side) {
                    CUDA_TRY(cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking));
                    CUDA_TRY(cudaStreamCreateWithFlags(&c->side_rest, cudaStreamNonBlocking));
                    CUDA_TRY(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
                    CUDA_TRY(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
                    CUDA_TRY(cudaEventCreateWithFlags(&c->ev_join_rest, cudaEventDisableTiming));
                    CUDA_TRY(cudaMalloc(&c->d_ws2, sizeof(unsigned long long) * 2 * 1024));
                    CUDA_TRY(cudaMemset(c->d_ws2, 0, sizeof(unsigned long long) * 2 * 1024));
                    CUDA_TRY(cudaMalloc(&c->d_ticket2, 64));
                    CUDA_TRY(cudaMemset(c->d_ticket2, 0, 64));
                    CUDA_TRY(cudaDeviceSynchronize());
                }
                CUDA_TRY(cudaEventRecord(c->ev_fork, (cudaStream_t)stream));
                CUDA_TRY(cudaStreamWaitEvent(c->side, c->ev_fork, 0));
                CUDA_TRY(cudaStreamWaitEvent(c->side_rest, c->ev_fork, 0));
                tcs = c->side; tws = c->d_ws2; ttk = c->d_ticket2;
            }
            int ti = 0;
            for (size_t q = 0; q < pl.prods.size(); ++q) {
                const SplitTerm &st = pl.prods[q];
                const up_column &ca = cols[st.col_a], &cb = cols[st.col_b];
                if (!pl.cc_kernels[q]) {
                    auto tc = ca.layout == UP_LAYOUT_QUADS ? upk_launch_contract_tq : upk_launch_contract_tc;
                    CUDA_TRY(tc(ca.data, ca.ld, ca.limbs, cb.data, cb.ld, cb.limbs, cols[0].n, st.sign, tws, ttk,
                                c->d_parts + (size_t)ti++ * LAs, LAs, c->num_sms, tcs));
                    c->launches++;
                    continue;
                }
                P.result = c->d_parts + (size_t)ti++ * LAs;
                if (up_status s = launch(c, pl.cc_kernels[q], P, P.n, (cudaStream_t)stream)) return s;
            }
            if (pl.rest_kernel) {
                P.result = c->d_parts + (size_t)ti++ * LAs;
                // (no programmatic launch beside the contraction: measured slower, r02_s67)
                if (up_status s = launch(c, pl.rest_kernel, P, P.n, overlap ? c->side_rest : (cudaStream_t)stream, !overlap))
                    return s;
            }
            if (overlap) {
                CUDA_TRY(cudaEventRecord(c->ev_join, c->side));
                CUDA_TRY(cudaEventRecord(c->ev_join_rest, c->side_rest));
                CUDA_TRY(cudaStreamWaitEvent((cudaStream_t)stream, c->ev_join, 0));
                CUDA_TRY(cudaStreamWaitEvent((cudaStream_t)stream, c->ev_join_rest, 0));
            }
            if (pl.rest_kernel && pl.rest_scale > 0) {
                const uint32_t *d_sc = nullptr;
                if (up_status s = pow10_device(c, pl.rest_scale, &d_sc)) return s;
                CUDA_TRY(upk_launch_combine_scaled(c->d_parts, T, LAs, d_partial, T - 1, d_sc,
                                                   limbs_for_precision(pl.rest_scale), (cudaStream_t)stream));
            } else {
                CUDA_TRY(upk_launch_combine(c->d_parts, T, LAs, d_partial, (cudaStream_t)stream));
            }
            c->launches++;
            return UP_OK;
        }
    }
    if (up_status s = expr_kernel(c, expr, cols, ncols, true, N, &k, &LA, nullptr, t)) return s;
    up_kparams P;
    fill_cols(P, cols, ncols);
    P.ws = c->d_ws;
    P.ticket = c->d_ticket;
    P.result = d_partial;
    P.flags = c->d_flags;
    return launch(c, k, P, P.n, (cudaStream_t)stream);
}

up_status up_sum(up_ctx *c, const up_column *col, int64_t n_global, uint32_t *d_partial, void *stream) {
    return up_sum_expr(c, "c1", col, 1, n_global, d_partial, stream);
}

up_status up_sum_combine(up_ctx *c, const uint32_t *d_partials, int32_t nranks, int32_t la, uint32_t *d_out,
                         void *stream) {
    if (!c || !d_partials || !d_out || nranks < 1 || la < 1) return fail(UP_E_INVAL, "bad combine arguments");
    CUDA_TRY(upk_launch_combine(d_partials, nranks, la, d_out, (cudaStream_t)stream));
    c->launches++;
    return UP_OK;
}

up_status up_check(up_ctx *c, void *stream) {
    if (!c) return fail(UP_E_INVAL, "null ctx");
    CUDA_TRY(cudaStreamSynchronize((cudaStream_t)stream));
    uint32_t f = 0;
    CUDA_TRY(cudaMemcpy(&f, c->d_flags, sizeof f, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemset(c->d_flags, 0, sizeof f));
    if (f & 1u) return fail(UP_E_OVERFLOW, "a value exceeded its inferred DECIMAL type");
    if (f & 2u) return fail(UP_E_DIVZERO, "division or modulo by zero");
    if (f & 4u) return fail(UP_E_RANGE, "an input value exceeds its DECIMAL(p,s)");
    if (f & 8u) return fail(UP_E_INVAL, "invalid input value (e.g. negative modexp base)");
    return UP_OK;
}

up_status up_format_decimal(const uint32_t *limbs, int32_t nlimbs, int32_t s, char *buf, size_t len) {
    if (!limbs || nlimbs < 1 || !buf || s < 0) return fail(UP_E_INVAL, "bad format arguments");
    HBig m;
    m.w.assign(limbs, limbs + nlimbs);
    const bool ng = (limbs[nlimbs - 1] >> 31) != 0;
    if (ng) {   // magnitude of a two's-complement value
        uint64_t cy = 1;
        for (auto &x : m.w) { uint64_t t = (uint64_t)(~x) + cy; x = (uint32_t)t; cy = t >> 32; }
    }
    m.trim();
    std::string d = m.to_dec();
    std::string out = (ng && !m.is_zero()) ? "-" : "";
    if (s == 0) out += d;
    else {
        if ((int)d.size() <= s) d = std::string((size_t)(s + 1 - (int)d.size()), '0') + d;
        out += d.substr(0, d.size() - (size_t)s) + "." + d.substr(d.size() - (size_t)s);
    }
    if (out.size() + 1 > len) return fail(UP_E_NOMEM, "buffer too small (%zu needed)", out.size() + 1);
    memcpy(buf, out.c_str(), out.size() + 1);
    return UP_OK;
}

// ---- grouped aggregation (NEXT-4): typing P:L1069-1080
}  // extern "C"
namespace {

struct AggPlan {
    std::vector<Typed> typed;
    std::vector<std::unique_ptr<Node>> opt;
    std::vector<AggItem> items;
    std::vector<ColType> types;
    long long words = 0;   // packed output words
    int mm_words = 0;      // MIN/MAX words per group record
    std::string key;
};

// result type of one aggregate over N tuples
up_status agg_result_type(int kind, const Node *root, long long N, int &p, int &s, int &LA) {
    const int ps = sum_precision(root->p, N);   // SUM: p + ceil(log10 N)
    LA = 0;
    switch (kind) {
    case AGG_SUM: p = ps; s = root->s; LA = limbs_for_precision(ps); return UP_OK;
    case AGG_MIN: case AGG_MAX: p = root->p; s = root->s; return UP_OK;
    case AGG_AVG: {
        // SUM rule, then the division rule with the divisor DECIMAL(ceil(log10 N)+1, 0):
        // (p1 - p2 + s2 + 5, s1 + 4)
        const int pd = (ps - root->p) + 1, sd = 0;
        p = ps - pd + sd + 5;
        s = root->s + 4;
        LA = limbs_for_precision(ps);
        return UP_OK;
    }
    default: return fail(UP_E_INVAL, "unknown aggregate kind %d", kind);
    }
}

up_status agg_plan(int32_t n_aggs, const int32_t *kinds, const char *const *exprs, const up_column *cols, int ncols,
                   long long N, int G, AggPlan &pl) {
    if (n_aggs < 1 || n_aggs > 32 || !kinds || !exprs) return fail(UP_E_INVAL, "need 1..32 aggregates");
    if (G < 1) return fail(UP_E_INVAL, "n_groups must be >= 1");
    pl.typed.resize((size_t)n_aggs);
    pl.key = "gagg|" + std::to_string(G) + "|" + std::to_string(N);
    for (int i = 0; i < ncols; ++i) pl.key += "|" + std::to_string(cols[i].p) + "," + std::to_string(cols[i].s);
    if (getenv("UP_NO_OPT")) pl.key += "|noopt";
    for (int a = 0; a < n_aggs; ++a) {
        Typed &t = pl.typed[(size_t)a];
        if (up_status st = type_expr(exprs[a], cols, ncols, t)) return st;
        if (a == 0) pl.types = t.types;
        int p = 0, s = 0, LA = 0;
        if (up_status st = agg_result_type(kinds[a], t.root.get(), N, p, s, LA)) return st;
        std::unique_ptr<Node> o = getenv("UP_NO_OPT") ? nullptr : optimize(t.root.get(), t.types);
        const Node *r = o ? o.get() : t.root.get();
        pl.opt.push_back(std::move(o));
        AggItem it;
        it.kind = kinds[a];
        it.root = r;
        it.LA = LA;
        it.Lr = limbs_for_precision(p);
        it.off = pl.words;
        pl.words += (long long)G * it.Lr;
        if (it.kind == AGG_MIN || it.kind == AGG_MAX) pl.mm_words += r->L;
        pl.items.push_back(it);
        pl.key += "|" + std::to_string(kinds[a]) + ":" + exprs[a];
    }
    return UP_OK;
}

}  // namespace
extern "C" {

up_status up_agg_type(const char *expr, int32_t kind, const up_column *cols, int ncols, int64_t n_global, int32_t *p,
                      int32_t *s, int32_t *limbs) {
    Typed t;
    if (up_status st = type_expr(expr, cols, ncols, t)) return st;
    const long long N = n_global > 0 ? n_global : (ncols ? cols[0].n : 0);
    int pp = 0, ss = 0, LA = 0;
    if (up_status st = agg_result_type(kind, t.root.get(), N, pp, ss, LA)) return st;
    if (p) *p = pp;
    if (s) *s = ss;
    if (limbs) *limbs = limbs_for_precision(pp);
    return UP_OK;
}

up_status up_eval_tpi(up_ctx *c, const char *op, const up_column *a, const up_column *b, int32_t tpi, int32_t div_algo,
                      up_column *out, void *stream) {
    if (!c || !op || !a || !b || !out) return fail(UP_E_INVAL, "need a ctx, an operator, two columns and out");
    int o = -1;
    if (!strcmp(op, "+")) o = 0;
    if (!strcmp(op, "-")) o = 1;
    if (!strcmp(op, "*")) o = 2;
    if (!strcmp(op, "/")) o = 3;
    if (o < 0) return fail(UP_E_INVAL, "operator must be + - * /");
    if (div_algo != 0 && div_algo != 1) return fail(UP_E_INVAL, "div_algo must be 0 (long division) or 1 (Newton-Raphson)");
    const up_column cols[2] = {*a, *b};
    for (int i = 0; i < 2; ++i) {
        if (up_status s = check_column(&cols[i], "input")) return s;
        if (cols[i].layout == UP_LAYOUT_QUADS) return fail(UP_E_UNSUPPORTED, "tpi inputs: limb planes or compact rows");
    }
    if (a->n != b->n) return fail(UP_E_INVAL, "columns differ in length");
    if (up_status s = check_column(out, "out")) return s;
    if (out->layout != UP_LAYOUT_PLANES) return fail(UP_E_UNSUPPORTED, "out must be limb planes");
    const std::string expr = std::string("c1") + op + "c2";
    Typed t;
    if (up_status s = type_expr(expr.c_str(), cols, 2, t)) return s;
    if (out->p != t.root->p || out->s != t.root->s || out->n != a->n)
        return fail(UP_E_INVAL, "out must be DECIMAL(%d,%d) with the inputs' rows", t.root->p, t.root->s);
    if (o == 3 && (t.root->l->L > 64 || t.root->r->L > 64 || t.root->L > 64))
        return fail(UP_E_UNSUPPORTED, "tpi division: operands up to 64 limbs");
    std::lock_guard<std::mutex> g(c->mu);
    std::string key = "tpi|" + expr + "|" + std::to_string(tpi) + "|" + std::to_string(div_algo);
    for (int i = 0; i < 2; ++i)
        key += "|" + std::to_string(cols[i].p) + "," + std::to_string(cols[i].s) + (cols[i].layout ? "c" : "");
    JitKernel *k = nullptr;
    std::string err;
    TpiInfo ti;
    if (up_status s = kernel_for(c, key, [&](GenInfo &info) {
            std::string src = gen_tpi_kernel(o, t.types[0], t.types[1], t.root.get(), tpi, div_algo == 1, ti, err);
            info.threads = 256;
            info.dyn_smem = ti.dyn_smem;
            return src; }, &k))
        return err.empty() ? s : fail(UP_E_UNSUPPORTED, "%s", err.c_str());
    up_kparams P;
    fill_cols(P, cols, 2);
    P.flags = c->d_flags;
    P.out = out->data;
    P.ld_out = out->ld;
    if (P.n == 0) return UP_OK;
    return launch(c, k, P, P.n * (long long)tpi, (cudaStream_t)stream);
}

up_status up_group_combine(up_ctx *c, int32_t n_aggs, const int32_t *kinds, const char *const *exprs,
                           const up_column *cols, int ncols, int32_t n_groups, int64_t n_global, const uint32_t *d_parts,
                           int32_t nranks, const uint64_t *d_counts, uint32_t *d_out, uint64_t *d_counts_out,
                           void *stream) {
    if (!c || !cols || ncols < 1 || !d_parts || !d_counts || !d_out || nranks < 1)
        return fail(UP_E_INVAL, "need a ctx, columns, partials, counts and d_out");
    if (n_aggs < 1 || n_aggs > 32 || !kinds) return fail(UP_E_INVAL, "need 1..32 aggregates");
    const long long N = n_global > 0 ? n_global : cols[0].n;
    std::vector<int32_t> pk((size_t)n_aggs);
    for (int a = 0; a < n_aggs; ++a) pk[(size_t)a] = kinds[a] == AGG_AVG ? AGG_SUM : kinds[a];
    AggPlan pp, pf;
    if (up_status s = agg_plan(n_aggs, pk.data(), exprs, cols, ncols, N, n_groups, pp)) return s;
    if (up_status s = agg_plan(n_aggs, kinds, exprs, cols, ncols, N, n_groups, pf)) return s;
    struct Desc { int kind, Lp, Lr, pad; long long poff, roff; };
    std::vector<Desc> d((size_t)n_aggs);
    for (int a = 0; a < n_aggs; ++a) {
        d[(size_t)a] = {kinds[a], pp.items[(size_t)a].Lr, pf.items[(size_t)a].Lr, 0, pp.items[(size_t)a].off,
                        pf.items[(size_t)a].off};
        if (d[(size_t)a].Lp > 80) return fail(UP_E_UNSUPPORTED, "group_combine: aggregate wider than 80 limbs");
    }
    cudaStream_t st = (cudaStream_t)stream;
    std::lock_guard<std::mutex> g(c->mu);
    if (up_status s = ensure_stage(c, sizeof(Desc) * d.size(), st)) return s;
    CUDA_TRY(cudaMemcpyAsync(c->d_stage, d.data(), sizeof(Desc) * d.size(), cudaMemcpyHostToDevice, st));
    CUDA_TRY(upk_launch_group_combine(d_parts, nranks, pp.words, (const unsigned long long *)d_counts, n_groups, n_aggs,
                                      c->d_stage, d_out, (unsigned long long *)d_counts_out, st));
    c->launches++;
    return UP_OK;
}

up_status up_group_aggregate(up_ctx *c, int32_t n_aggs, const int32_t *kinds, const char *const *exprs,
                             const up_column *cols, int ncols, const int32_t *d_group, int32_t n_groups,
                             int64_t n_global, uint32_t *d_out, uint64_t *d_counts, void *stream) {
    if (!c || !cols || ncols < 1 || !d_out || !d_counts) return fail(UP_E_INVAL, "need a ctx, columns, d_out and d_counts");
    for (int i = 0; i < ncols; ++i) {
        if (up_status s = check_column(&cols[i], "input")) return s;
        if (up_status s = need_planes(&cols[i], "group_aggregate input")) return s;
        if (cols[i].n != cols[0].n) return fail(UP_E_INVAL, "columns differ in length");
    }
    if (!d_group && n_groups != 1) return fail(UP_E_INVAL, "d_group == NULL needs n_groups == 1");
    if ((uintptr_t)d_group & 15) return fail(UP_E_INVAL, "d_group must be 16-byte aligned device memory");
    const long long N = n_global > 0 ? n_global : cols[0].n;
    if (N < cols[0].n) return fail(UP_E_INVAL, "n_global < local rows");
    AggPlan pl;
    if (up_status s = agg_plan(n_aggs, kinds, exprs, cols, ncols, N, n_groups, pl)) return s;
    std::lock_guard<std::mutex> g(c->mu);
    JitKernel *k = nullptr;
    int mmw = 0;
    if (up_status s = kernel_for(c, pl.key, [&](GenInfo &info) {
            std::string src = gen_group_agg_kernel(pl.items, pl.types, n_groups, info, mmw);
            if (info.dyn_smem > 200 * 1024) { fail(UP_E_UNSUPPORTED, "too many groups for one block's records"); return std::string(); }
            return src; }, &k))
        return s;
    up_kparams P;
    fill_cols(P, cols, ncols);
    P.ws = c->d_ws;
    P.ticket = c->d_ticket;
    P.flags = c->d_flags;
    P.result = d_out;
    P.group = d_group;
    P.counts = (unsigned long long *)d_counts;
    if (pl.mm_words) {
        const long long want = (P.n + k->threads - 1) / k->threads;
        const long long grid = std::max(1ll, std::min(want, (long long)k->blocks_per_sm * c->num_sms));
        void *sp = nullptr;
        const size_t bytes = (size_t)grid * (size_t)n_groups * (size_t)pl.mm_words * 4;
        if (bytes > c->scratch_bytes) {
            if (c->d_scratch) { CUDA_TRY(cudaDeviceSynchronize()); CUDA_TRY(cudaFree(c->d_scratch)); c->d_scratch = nullptr; }
            CUDA_TRY(cudaMalloc(&c->d_scratch, bytes));
            c->scratch_bytes = bytes;
        }
        sp = c->d_scratch;
        P.scratch = (unsigned int *)sp;
    }
    return launch(c, k, P, std::max(P.n, 1ll), (cudaStream_t)stream);
}

up_status up_gen_group_agg_source(int32_t n_aggs, const int32_t *kinds, const char *const *exprs, const up_column *cols,
                                  int ncols, int32_t n_groups, int64_t n_global, char *buf, size_t len) {
    AggPlan pl;
    const long long N = n_global > 0 ? n_global : (ncols ? cols[0].n : 0);
    if (up_status s = agg_plan(n_aggs, kinds, exprs, cols, ncols, N, n_groups, pl)) return s;
    GenInfo info;
    int mmw = 0;
    std::string src = gen_group_agg_kernel(pl.items, pl.types, n_groups, info, mmw);
    if (!buf || src.size() + 1 > len) return fail(UP_E_NOMEM, "need %zu bytes", src.size() + 1);
    memcpy(buf, src.c_str(), src.size() + 1);
    return UP_OK;
}

// ---- diagnostics (no GPU needed): generated source and an NVRTC-only compile
up_status up_gen_tpi_source(const char *op, const up_column *cols, int32_t tpi, int32_t div_algo, char *buf, size_t len) {
    if (!op || !cols) return fail(UP_E_INVAL, "null argument");
    const int o = !strcmp(op, "+") ? 0 : !strcmp(op, "-") ? 1 : !strcmp(op, "*") ? 2 : !strcmp(op, "/") ? 3 : -1;
    if (o < 0) return fail(UP_E_INVAL, "operator must be + - * /");
    const std::string expr = std::string("c1") + op + "c2";
    Typed t;
    if (up_status s = type_expr(expr.c_str(), cols, 2, t)) return s;
    TpiInfo ti;
    std::string err;
    const std::string src = gen_tpi_kernel(o, t.types[0], t.types[1], t.root.get(), tpi, div_algo == 1, ti, err);
    if (src.empty()) return fail(UP_E_UNSUPPORTED, "%s", err.c_str());
    if (src.size() + 1 > len) return fail(UP_E_NOMEM, "buffer too small");
    memcpy(buf, src.c_str(), src.size() + 1);
    return UP_OK;
}

up_status up_gen_source(const char *variant, const char *expr, const up_column *cols, int ncols, int64_t n_global,
                        char *buf, size_t len) {
    if (!variant || !buf) return fail(UP_E_INVAL, "null argument");
    Typed t;
    if (up_status s = type_expr(expr, cols, ncols, t)) return s;
    GenOpts o;
    o.sum = strcmp(variant, "sum") == 0;
    const long long N = n_global > 0 ? n_global : (ncols ? cols[0].n : 0);
    o.LA = o.sum ? limbs_for_precision(sum_precision(t.root->p, N)) : 0;
    GenInfo info;
    std::string src;
    std::unique_ptr<Node> opt_root = getenv("UP_NO_OPT") ? nullptr : optimize(t.root.get(), t.types);
    const Node *gen_root = opt_root ? opt_root.get() : t.root.get();
    bool any_compact = false;   // as expr_kernel: the wide regime reads limb planes only
    for (const ColType &ct : t.types) any_compact = any_compact || ct.Lb > 0 || ct.Q;
    if (o.sum && !any_compact && max_limbs(gen_root) >= kWideMinLimbs && o.LA <= 512 && !getenv("UP_NO_WIDE"))
        src = gen_wide_sum_kernel(gen_root, t.types, o.LA, info);
    if (src.empty()) src = gen_expr_kernel(gen_root, t.types, o, info);
    if (src.size() + 1 > len) return fail(UP_E_NOMEM, "need %zu bytes", src.size() + 1);
    memcpy(buf, src.c_str(), src.size() + 1);
    return UP_OK;
}

up_status up_nvrtc_compile(const char *src, const char *cubin_path, char *log, size_t len) {
    nvrtcProgram prog;
    const char *hdrs[3] = {k_up_dev_src, k_up_kparams_src, k_up_wide_src};
    const char *names[3] = {"up_dev.cuh", "up_kparams.h", "up_wide.cuh"};
    if (nvrtcCreateProgram(&prog, src, "upk.cu", 3, hdrs, names) != NVRTC_SUCCESS)
        return fail(UP_E_NVRTC, "nvrtcCreateProgram failed");
    std::vector<const char *> opts(kNvrtcOpts, kNvrtcOpts + sizeof kNvrtcOpts / sizeof kNvrtcOpts[0]);
    opts.push_back("-Xptxas=-v");
    nvrtcResult r = nvrtcCompileProgram(prog, (int)opts.size(), opts.data());
    size_t ls = 0;
    nvrtcGetProgramLogSize(prog, &ls);
    std::string lg(ls, '\0');
    nvrtcGetProgramLog(prog, &lg[0]);
    if (log && len) { size_t k = std::min(len - 1, lg.size()); memcpy(log, lg.data(), k); log[k] = 0; }
    if (r != NVRTC_SUCCESS) { nvrtcDestroyProgram(&prog); return fail(UP_E_NVRTC, "NVRTC: %s", nvrtcGetErrorString(r)); }
    if (cubin_path) {
        size_t cs = 0;
        nvrtcGetCUBINSize(prog, &cs);
        std::vector<char> cubin(cs);
        nvrtcGetCUBIN(prog, cubin.data());
        std::ofstream(cubin_path, std::ios::binary).write(cubin.data(), (std::streamsize)cs);
    }
    nvrtcDestroyProgram(&prog);
    return UP_OK;
}

// Canonical text of the optimised tree (alignment scheduling + constant folding)
up_status up_expr_optimized(const char *expr, const up_column *cols, int ncols, char *buf, size_t len) {
    Typed t;
    if (up_status s = type_expr(expr, cols, ncols, t)) return s;
    auto o = optimize(t.root.get(), t.types);
    std::string txt = canonical(o.get()) + " : (" + std::to_string(o->p) + "," + std::to_string(o->s) + ")";
    if (txt.size() + 1 > len) return fail(UP_E_NOMEM, "buffer too small");
    memcpy(buf, txt.c_str(), txt.size() + 1);
    return UP_OK;
}

// generated row-contraction source (diagnostics / prewarm)
up_status up_gen_contract_source(int32_t La, int32_t Lb, int32_t LA, int sign, char *buf, size_t len) {
    GenInfo info;
    const std::string src = gen_contract_kernel(La, Lb, LA, sign, 0, 1, info);
    if (src.empty()) return fail(UP_E_UNSUPPORTED, "no contraction kernel");
    if (src.size() + 1 > len) return fail(UP_E_NOMEM, "buffer too small");
    memcpy(buf, src.c_str(), src.size() + 1);
    return UP_OK;
}

// Fill the on-disk cubin cache for a source (no GPU needed).
up_status up_jit_prewarm(const char *src) {
    if (!src) return fail(UP_E_INVAL, "null source");
    const std::string cpath = cache_path(src);
    std::vector<char> cubin;
    if (cpath.empty()) return fail(UP_E_INVAL, "no cache directory");
    if (read_file(cpath, cubin)) return UP_OK;
    if (up_status st = nvrtc_to_cubin(src, cubin)) return st;
    write_file_atomic(cpath, cubin);
    return UP_OK;
}

// modexp / sin_taylor live in special.cpp
}  // extern "C"

// exported to special.cpp
up_status up_internal_compile(up_ctx *c, const std::string &src, int rows_per_thread, int ws_slots, int threads,
                              void **fn_out, int *blocks_per_sm, int dyn_smem) {
    JitKernel *k = nullptr;
    up_status s = compile(c, src, &k);
    if (s) return s;
    k->rows_per_thread = rows_per_thread;
    k->ws_slots = ws_slots;
    if (threads != k->threads || dyn_smem != k->dyn_smem) {
        k->threads = threads;
        if (dyn_smem > 0)
            CU_TRY(drv.FuncSetAttribute(k->fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, dyn_smem));
        k->dyn_smem = dyn_smem;
        int nb = 0;
        CU_TRY(drv.OccupancyMaxActiveBlocksPerMultiprocessor(&nb, k->fn, threads, (size_t)dyn_smem));
        k->blocks_per_sm = std::max(1, nb);
    }
    *fn_out = k;
    if (blocks_per_sm) *blocks_per_sm = k->blocks_per_sm;
    return UP_OK;
}
up_status up_internal_launch(up_ctx *c, void *kp, up_kparams &P, long long work_items, cudaStream_t st) {
    return launch(c, (JitKernel *)kp, P, work_items, st);
}
std::mutex &up_internal_mutex(up_ctx *c) { return c->mu; }
unsigned long long *up_internal_ws(up_ctx *c) { return c->d_ws; }
uint32_t *up_internal_ticket(up_ctx *c) { return c->d_ticket; }
uint32_t *up_internal_flags(up_ctx *c) { return c->d_flags; }
int up_internal_num_sms(up_ctx *c) { return c->num_sms; }
up_status up_internal_scratch(up_ctx *c, size_t bytes, void **out);
up_status scratch_locked(up_ctx *c, size_t bytes, void **out) { return up_internal_scratch(c, bytes, out); }
up_status up_internal_scratch(up_ctx *c, size_t bytes, void **out) {
    if (bytes > c->scratch_bytes) {
        if (c->d_scratch) {
            CUDA_TRY(cudaDeviceSynchronize());
            CUDA_TRY(cudaFree(c->d_scratch));
            c->d_scratch = nullptr;
        }
        CUDA_TRY(cudaMalloc(&c->d_scratch, bytes));
        c->scratch_bytes = bytes;
    }
    *out = c->d_scratch;
    return UP_OK;
}
up_status up_internal_fail(up_status st, const std::string &msg) { return fail(st, "%s", msg.c_str()); }

void up_internal_add_launches(up_ctx *c, long long k) {
    if (c) c->launches += (uint64_t)k;
}
