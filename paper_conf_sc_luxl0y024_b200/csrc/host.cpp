// host.cpp -- the C-ABI library (include/smiless.h): validation, derived tables, NVRTC
// specialisation of the evaluator per (DAG, window grid, range mode), launches, result
// decode.  SURVEY 8(a) steps a1-a10 on the host side; every per-candidate computation
// runs in the CUDA kernels (evaluator.cuh via NVRTC, kernels.cu via nvcc).
//
// No CPU fallback: without a device, driver or NVRTC the calls fail with
// SMILESS_ECUDA / SMILESS_EJIT.
#include "smiless.h"

#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvrtc.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <functional>
#include <map>
#include <memory>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "kernels.h"
#include <nvtx3/nvToolsExt.h>

extern "C" const char smiless_evaluator_src[];  // generated from evaluator.cuh at build time

namespace {

typedef long long i64;
typedef unsigned long long u64;

// ------------------------------------------------------------------------------------
// Dynamically resolved NVRTC and CUDA driver entry points (so that the library loads on
// a host without a GPU; nothing here runs until the first plan/evaluate).
// ------------------------------------------------------------------------------------
struct NvrtcApi {
    bool ok = false;
    std::string why;
    decltype(&nvrtcCreateProgram) create = nullptr;
    decltype(&nvrtcCompileProgram) compile = nullptr;
    decltype(&nvrtcGetProgramLogSize) log_size = nullptr;
    decltype(&nvrtcGetProgramLog) get_log = nullptr;
    decltype(&nvrtcGetCUBINSize) cubin_size = nullptr;
    decltype(&nvrtcGetCUBIN) get_cubin = nullptr;
    decltype(&nvrtcDestroyProgram) destroy = nullptr;
    decltype(&nvrtcGetErrorString) err_str = nullptr;
};

NvrtcApi &nvrtc() {
    static NvrtcApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *env = getenv("SMILESS_NVRTC");
        // the toolkit's own NVRTC first: a bare soname may resolve to an older copy another
        // library (e.g. a framework's bundled runtime) already loaded into the process
        const char *cands[] = {env, "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so.12", "libnvrtc.so"};
        void *h = nullptr;
        for (const char *c : cands) {
            if (!c) continue;
            h = dlopen(c, RTLD_NOW | RTLD_LOCAL);
            if (h) break;
        }
        if (!h) {
            api.why = "cannot dlopen libnvrtc.so.12";
            return;
        }
#define SMILESS_SYM(field, name)                                       \
    api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name)); \
    if (!api.field) { api.why = std::string("missing NVRTC symbol ") + name; return; }
        SMILESS_SYM(create, "nvrtcCreateProgram");
        SMILESS_SYM(compile, "nvrtcCompileProgram");
        SMILESS_SYM(log_size, "nvrtcGetProgramLogSize");
        SMILESS_SYM(get_log, "nvrtcGetProgramLog");
        SMILESS_SYM(cubin_size, "nvrtcGetCUBINSize");
        SMILESS_SYM(get_cubin, "nvrtcGetCUBIN");
        SMILESS_SYM(destroy, "nvrtcDestroyProgram");
        SMILESS_SYM(err_str, "nvrtcGetErrorString");
#undef SMILESS_SYM
        api.ok = true;
    });
    return api;
}

struct DriverApi {
    bool ok = false;
    std::string why;
    CUresult (*moduleLoadData)(CUmodule *, const void *) = nullptr;
    CUresult (*moduleUnload)(CUmodule) = nullptr;
    CUresult (*moduleGetFunction)(CUfunction *, CUmodule, const char *) = nullptr;
    CUresult (*funcSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
    CUresult (*funcGetAttribute)(int *, CUfunction_attribute, CUfunction) = nullptr;
    CUresult (*launchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                             CUstream, void **, void **) = nullptr;
    CUresult (*occupancy)(int *, CUfunction, int, size_t) = nullptr;
    CUresult (*getErrorString)(CUresult, const char **) = nullptr;
};

DriverApi &driver() {
    static DriverApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        auto get = [&](const char *name, void **fn) -> bool {
            cudaDriverEntryPointQueryResult q;
            cudaError_t e = cudaGetDriverEntryPointByVersion(name, fn, 12000, cudaEnableDefault, &q);
            if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !*fn) {
                api.why = std::string("cannot resolve driver entry point ") + name;
                return false;
            }
            return true;
        };
        if (!get("cuModuleLoadData", (void **)&api.moduleLoadData)) return;
        if (!get("cuModuleUnload", (void **)&api.moduleUnload)) return;
        if (!get("cuModuleGetFunction", (void **)&api.moduleGetFunction)) return;
        if (!get("cuFuncSetAttribute", (void **)&api.funcSetAttribute)) return;
        if (!get("cuFuncGetAttribute", (void **)&api.funcGetAttribute)) return;
        if (!get("cuLaunchKernel", (void **)&api.launchKernel)) return;
        if (!get("cuOccupancyMaxActiveBlocksPerMultiprocessor", (void **)&api.occupancy)) return;
        if (!get("cuGetErrorString", (void **)&api.getErrorString)) return;
        api.ok = true;
    });
    return api;
}

// ------------------------------------------------------------------------------------
// Kernel parameter block: must match PlanParams in evaluator.cuh byte for byte.
// ------------------------------------------------------------------------------------
struct PlanParamsHost {
    const int *tabI;
    const int *tabT;
    const double *tabU;
    const void *off;
    const i64 *scal;
    u64 *counter;
    u64 *stats;
    u64 *blk_best;
    u64 unit_begin, unit_end;
    u64 cand_begin, cand_end;
    u64 claims_end;
    u64 claims_begin;
    i64 n_steps;
    i64 n_off;
    int sumM;
    int sla;
    int prune;
    int shard, n_shards;
    int chunk_units;
    double *dump;
    const int *tabNI;
    int zero;
    const u64 *list_in;
    const unsigned *list_n;
    u64 list_upp;
    u64 *list_out;
    unsigned *list_cnt;
    u64 list_base;
    i64 horizon;
    int slas[8];
    const int *tabW;               // [sumM] per-row windows (SM_ROWWIN) or a dummy table
    u64 *inc;                      // incumbent cost bits (cost-bound pruning)
    const i64 *rrem;               // [chunks] r_{J-1} - r_{(q+1)K}
    u64 cap;                       // cost cap bits (~0: none)
    int cost_prune;
    int no_count;                  // 1: the units were counted by an earlier pass
    u64 list_in_cap;               // list mode: entries list_in holds (clamps *list_n)
    int fixed[SMILESS_MAX_FUNCS];  // evaluator uses SM_NFIXED_ALLOC <= SMILESS_MAX_FUNCS; extra tail is ignored
};

// Mirror of MemoParams (evaluator.cuh, prefix memoisation kernels).
struct MemoParamsHost {
    const int *tabNI, *tabT, *tabW;
    const double *tabU;
    const void *off;
    const i64 *scal;
    u64 *counter;
    u64 *stats;
    u64 *blk_best;
    void *xbuf;
    void *rec_nx;
    double *rec_pre;
    void *rec_nlu;
    double *dump;
    u64 pref_begin, pref_end;
    u64 unit_begin, unit_end;
    u64 cand_begin, cand_end;
    i64 n_steps;
    i64 n_off;
    int sumM;
    int sla;
    int zero;
    int slas[8];
    u64 *cost_list;                // split cost: units holding a feasible candidate
    unsigned *cost_n;
    int shard, n_shards;           // fused kernel: tile c belongs to shard c % n_shards
    int fixed[SMILESS_MAX_FUNCS];
};

// Mirror of BoundParams (evaluator.cuh, B&B pre-pass kernel).
struct BoundParamsHost {
    const int *tabNI;
    const int *tabT;
    const void *off;
    u64 *counter;
    u64 *stats;
    u64 *list_out;
    unsigned *list_cnt;
    u64 prefix_begin, prefix_end;
    u64 cands_per_prefix;
    u64 cand_begin, cand_end;
    i64 n_steps;
    i64 n_off;
    int sumM;
    int sla;
    int prune_check;
    int zero;
    const u64 *list_in;
    const unsigned *list_n;
    u64 list_upp;
    int nimin[SMILESS_MAX_FUNCS];
    const int *tabW;
    const double *tabU;
    const i64 *scal;
    u64 *inc;                      // incumbent cost bits shared with the evaluator
    int cost_prune;
    int pad0;
    u64 list_stride, list_r0;      // list mode: prefix = list_in[c / upp] * stride + r0 + c % upp
    u64 list_cap;                  // capacity of list_out
    unsigned *overflow;            // set to 1 if a launch would exceed list_cap (never, by sizing)
    int shard, n_shards;           // ordinals c = c' * n_shards + shard of the launch
    int attr_shard, attr_n;        // replicated level: decided counted for c % attr_n == attr_shard
    u64 *list_key;                 // optional static cost lower bound per survivor (best-first order)
    int fixed[SMILESS_MAX_FUNCS];
};

// CTA size of the evaluator / bound kernels (SMILESS_THREADS tunes it; multiple of 32, <= 1024).
int threads_per_cta() {
    static const int t = [] {
        const char *e = getenv("SMILESS_THREADS");
        const int v = e ? atoi(e) : 256;
        return (v >= 64 && v <= 1024 && v % 32 == 0) ? v : 256;
    }();
    return t;
}
#define kThreads threads_per_cta()
// CTA size and min CTAs/SM of the memoised variants kernel.  2 x 256 threads (128 registers)
// measured best on C2 (profiles/r01f_sweep_variants.md; SMILESS_VTHREADS / SMILESS_VMINB tune it)
int vthreads_per_cta() {
    static const int t = [] {
        const char *e = getenv("SMILESS_VTHREADS");
        const int v = e ? atoi(e) : 256;
        return (v >= 64 && v <= 1024 && v % 32 == 0) ? v : 256;
    }();
    return t;
}
// L2 prefetch distance (4-step groups) of the variants kernel's x stream (SMILESS_XPF tunes it)
int xpf_groups() {
    const char *e = getenv("SMILESS_XPF");
    return e ? std::min(64, std::max(1, atoi(e))) : 8;
}

int vmin_blocks() {
    static const int b = [] {
        const char *e = getenv("SMILESS_VMINB");
        const int v = e ? atoi(e) : 2;
        return (v >= 1 && v <= 8) ? v : 2;
    }();
    return b;
}
constexpr int kChunkUnits = 256;     // sharding / claim granularity in units (multiple of 32)

struct JitKernel {
    CUmodule mod = nullptr;
    CUfunction fn = nullptr;
    CUfunction fn_bound = nullptr, fn_bound_a = nullptr, fn_up = nullptr, fn_var = nullptr, fn_varc = nullptr;
    CUfunction fn_fused = nullptr, fn_bound_m = nullptr;
    size_t smem_up = 0, smem_var = 0, smem_fused = 0;
    int blocks_up = 0, blocks_var = 0, blocks_fused = 0;
    size_t smem = 0, smem_bound = 0;
    int blocks_per_sm = 0, blocks_bound = 0;
    int regs = 0;
    size_t params_size = 0;
};

template <typename T>
struct DevBuf {
    T *p = nullptr;
    size_t n = 0;
    cudaError_t ensure(size_t want) {
        if (want <= n && p) return cudaSuccess;
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
        cudaError_t e = cudaMalloc((void **)&p, std::max<size_t>(want, 1) * sizeof(T));
        if (e == cudaSuccess) n = want;
        return e;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
};

}  // namespace

struct smiless_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    std::string err;

    // DAG
    int N = 0;
    std::vector<int32_t> pred_ptr, pred_idx;
    u64 sinkmask = 0;
    bool dag_loaded = false;

    // profiles
    std::vector<int32_t> M, row0;
    std::vector<int32_t> I, T;
    std::vector<double> U;
    int sumM = 0;
    i64 Tmax = 0, Imax = 0;
    bool prof_loaded = false;
    bool tables_dirty = true;

    // device state
    bool dev_ready = false;
    int n_sms = 0;
    DevBuf<int> dI, dNI, dT, dPtr, dIdx;
    DevBuf<double> dU;
    DevBuf<i64> dArr;
    DevBuf<unsigned char> dOff;
    DevBuf<i64> dScal;
    DevBuf<i64> dRrem;                       // real time left after each chunk (cost bound)
    DevBuf<int> dErr;
    DevBuf<u64> dCounter, dStats, dBlk, dIdxEval, dInc;
    DevBuf<double> dCost;
    DevBuf<i64> dLat;
    DevBuf<unsigned char> dFeas;
    DevBuf<double> dDump;
    DevBuf<u64> dList, dListA, dListM, dCostList, dListKeyA;
    DevBuf<unsigned> dCostN;
    DevBuf<unsigned> dListCnt, dListCntA, dListCntM, dChunkCnt, dChunkCntM;
    DevBuf<ResBlock> dDig;                   // smiless_plan_digits: each digit's winner
    DevBuf<int> dW;                          // per-row windows of the current plan (padded)
    DevBuf<unsigned char> dX;                // memoised last-function inputs [n_off/4][prefix][4]
    DevBuf<i64> dRecNx, dRecNlu;             // per-prefix records (int32 or int64 time)
    DevBuf<double> dRecPre;
    std::vector<int> hW;                     // host copy of what dW holds
    DevBuf<ResBlock> dRes;
    ResBlock *hRes = nullptr;    // pinned [SMILESS_MAX_SLAS]
    int nsla = 1;                // argmin keys of the plan being compiled (SLA sweep)
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};

    std::map<std::string, JitKernel> jit_cache;
    u64 h2d = 0, d2h = 0;        // host<->device bytes copied by the current plan call
};

namespace {

thread_local std::string g_create_err;

int fail(smiless_ctx *c, int code, const char *fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) c->err = buf;
    return code;
}

int cuda_fail(smiless_ctx *c, cudaError_t e, const char *what) {
    return fail(c, SMILESS_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

int drv_fail(smiless_ctx *c, CUresult r, const char *what) {
    const char *s = "?";
    if (driver().getErrorString) driver().getErrorString(r, &s);
    return fail(c, SMILESS_ECUDA, "%s: %s", what, s);
}

#define CK(expr, what)                                          \
    do {                                                        \
        cudaError_t e_ = (expr);                                \
        if (e_ != cudaSuccess) return cuda_fail(ctx, e_, what); \
    } while (0)

int ensure_device(smiless_ctx *ctx) {
    if (ctx->dev_ready) return SMILESS_OK;
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0) return fail(ctx, SMILESS_ECUDA, "no CUDA device: %s", cudaGetErrorString(e));
    if (ctx->device >= n) return fail(ctx, SMILESS_ECUDA, "device %d out of range (%d devices)", ctx->device, n);
    CK(cudaSetDevice(ctx->device), "cudaSetDevice");
    CK(cudaFree(nullptr), "context init");
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, ctx->device), "cudaGetDeviceProperties");
    if (prop.major != 10 || prop.minor != 0)
        return fail(ctx, SMILESS_ECUDA, "device %d is sm_%d%d; this library is built for sm_100a (B200)", ctx->device,
                    prop.major, prop.minor);
    ctx->n_sms = prop.multiProcessorCount;
    if (!driver().ok) return fail(ctx, SMILESS_ECUDA, "CUDA driver API: %s", driver().why.c_str());
    for (auto &ev : ctx->ev) CK(cudaEventCreate(&ev), "cudaEventCreate");
    CK(cudaMallocHost((void **)&ctx->hRes, sizeof(ResBlock) * SMILESS_MAX_SLAS), "cudaMallocHost");
    CK(ctx->dRes.ensure(SMILESS_MAX_SLAS), "cudaMalloc");
    CK(ctx->dScal.ensure(546), "cudaMalloc");         // [0] R, [1] o_last, [2..546) scale-out sums (prep_tail)
    CK(ctx->dErr.ensure(1), "cudaMalloc");
    CK(ctx->dCounter.ensure(1), "cudaMalloc");
    CK(ctx->dStats.ensure(2), "cudaMalloc");
    CK(ctx->dInc.ensure(1), "cudaMalloc");
    ctx->dev_ready = true;
    return SMILESS_OK;
}

int upload_tables(smiless_ctx *ctx) {
    if (!ctx->tables_dirty) return SMILESS_OK;
    // one spare all-zero row after the last (I = T = 0, U = 0): the virtual sink of
    // scale-out plans (see dag_spec_source), staged with sumM + 1 rows
    const size_t padI = (size_t)((ctx->sumM + 1 + 3) & ~3);
    const size_t padU = (size_t)((ctx->sumM + 1 + 1) & ~1);
    std::vector<int> I(padI, 0), NI(padI, 0), T(padI, 0);
    std::vector<double> U(padU, 0.0);
    std::copy(ctx->I.begin(), ctx->I.end(), I.begin());
    for (int r = 0; r < ctx->sumM; ++r) NI[r] = -ctx->I[r];
    std::copy(ctx->T.begin(), ctx->T.end(), T.begin());
    std::copy(ctx->U.begin(), ctx->U.end(), U.begin());
    CK(ctx->dI.ensure(padI), "cudaMalloc");
    CK(ctx->dNI.ensure(padI), "cudaMalloc");
    CK(ctx->dT.ensure(padI), "cudaMalloc");
    CK(ctx->dU.ensure(padU), "cudaMalloc");
    CK(ctx->dPtr.ensure(ctx->pred_ptr.size()), "cudaMalloc");
    CK(ctx->dIdx.ensure(std::max<size_t>(ctx->pred_idx.size(), 1)), "cudaMalloc");
    // stream-ordered uploads: the kernels that read them run on ctx->stream, which may be a
    // non-blocking stream (not ordered after the legacy default stream).  The pageable
    // sources are staged before cudaMemcpyAsync returns, so the local vectors may go.
    cudaStream_t st = ctx->stream;
    ctx->h2d += 3 * padI * sizeof(int) + padU * sizeof(double) + ctx->pred_ptr.size() * sizeof(int) +
                ctx->pred_idx.size() * sizeof(int);
    CK(cudaMemcpyAsync(ctx->dI.p, I.data(), padI * sizeof(int), cudaMemcpyHostToDevice, st), "H2D tables");
    CK(cudaMemcpyAsync(ctx->dNI.p, NI.data(), padI * sizeof(int), cudaMemcpyHostToDevice, st), "H2D tables");
    CK(cudaMemcpyAsync(ctx->dT.p, T.data(), padI * sizeof(int), cudaMemcpyHostToDevice, st), "H2D tables");
    CK(cudaMemcpyAsync(ctx->dU.p, U.data(), padU * sizeof(double), cudaMemcpyHostToDevice, st), "H2D tables");
    CK(cudaMemcpyAsync(ctx->dPtr.p, ctx->pred_ptr.data(), ctx->pred_ptr.size() * sizeof(int), cudaMemcpyHostToDevice,
                       st),
       "H2D dag");
    if (!ctx->pred_idx.empty())
        CK(cudaMemcpyAsync(ctx->dIdx.p, ctx->pred_idx.data(), ctx->pred_idx.size() * sizeof(int),
                           cudaMemcpyHostToDevice, st),
           "H2D dag");
    ctx->tables_dirty = false;
    return SMILESS_OK;
}

// ------------------------------------------------------------------------------------
// Argument validation and derived quantities
// ------------------------------------------------------------------------------------
bool space_size_of(const smiless_ctx *c, int W, int n_fixed, u64 *out) {
    unsigned __int128 s = 1;
    for (int k = n_fixed; k < c->N; ++k) {
        s *= (unsigned __int128)((u64)c->M[k] * (u64)W);
        if (s > ((unsigned __int128)1 << 63)) return false;   // indices 0 .. 2^63-1 fit int64
    }
    *out = (u64)s;
    return true;
}

int validate_args(smiless_ctx *ctx, const smiless_plan_args *a, bool need_arrivals_host_check) {
    if (!a) return fail(ctx, SMILESS_EINVAL, "args is NULL");
    if (!ctx->dag_loaded || !ctx->prof_loaded) return fail(ctx, SMILESS_ESTATE, "load_dag and load_profiles first");
    if (a->n_windows < 1 || a->n_windows > SMILESS_MAX_WINDOWS)
        return fail(ctx, SMILESS_EINVAL, "n_windows must be in [1, %d]", SMILESS_MAX_WINDOWS);
    if (!a->windows_us) return fail(ctx, SMILESS_EINVAL, "windows_us is NULL");
    for (int v = 0; v < a->n_windows; ++v) {
        if (a->windows_us[v] < 0 || a->windows_us[v] >= (1 << 29))
            return fail(ctx, SMILESS_EINVAL, "window %d out of [0, 2^29)", v);
        if (v && a->windows_us[v] <= a->windows_us[v - 1])
            return fail(ctx, SMILESS_EINVAL, "windows must be strictly increasing");
    }
    if (a->sla_us < 0 || a->sla_us >= (1ll << 29)) return fail(ctx, SMILESS_EINVAL, "sla_us out of [0, 2^29)");
    if (a->row_windows_us) {
        if (a->n_windows != 1) return fail(ctx, SMILESS_EINVAL, "row_windows_us requires n_windows == 1");
        for (int r = 0; r < ctx->sumM; ++r)
            if (a->row_windows_us[r] < 0 || a->row_windows_us[r] >= (1 << 29))
                return fail(ctx, SMILESS_EINVAL, "row window %d out of [0, 2^29)", r);
    }
    if (a->n_arrivals < 1) return fail(ctx, SMILESS_EINVAL, "n_arrivals must be >= 1");
    if (a->n_arrivals > (1ll << 31)) return fail(ctx, SMILESS_EINVAL, "n_arrivals too large");
    if (!a->arrivals_us) return fail(ctx, SMILESS_EINVAL, "arrivals_us is NULL");
    if (need_arrivals_host_check && !(a->flags & SMILESS_FLAG_ARRIVALS_ON_DEVICE)) {
        const i64 LIM = (i64)1 << 62;
        for (i64 j = 0; j < a->n_arrivals; ++j) {
            const i64 r = a->arrivals_us[j];
            if (r <= -LIM || r >= LIM) return fail(ctx, SMILESS_EINVAL, "arrival %lld out of range", (long long)j);
            if (j && r < a->arrivals_us[j - 1])
                return fail(ctx, SMILESS_EINVAL, "arrivals must be non-decreasing (index %lld)", (long long)j);
        }
    }
    if (a->n_fixed < 0 || a->n_fixed > ctx->N) return fail(ctx, SMILESS_EINVAL, "n_fixed out of [0, N]");
    if (a->n_fixed > 0 && !a->fixed_digits) return fail(ctx, SMILESS_EINVAL, "fixed_digits is NULL");
    for (int k = 0; k < a->n_fixed; ++k)
        if (a->fixed_digits[k] < 0 || (i64)a->fixed_digits[k] >= (i64)ctx->M[k] * a->n_windows)
            return fail(ctx, SMILESS_EINVAL, "fixed digit %d out of range", k);
    u64 space;
    if (!space_size_of(ctx, a->n_windows, a->n_fixed, &space))
        return fail(ctx, SMILESS_ERANGE, "candidate space exceeds 2^63-1; pin leading digits with n_fixed");
    if (a->n_shards < 0 || (a->n_shards > 0 && (a->shard < 0 || a->shard >= a->n_shards)))
        return fail(ctx, SMILESS_EINVAL, "bad shard/n_shards");
    if (a->instances)
        for (int k = 0; k < ctx->N; ++k)
            if (a->instances[k] < 1 || a->instances[k] > SMILESS_MAX_INSTANCES)
                return fail(ctx, SMILESS_EINVAL, "instances[%d] out of [1, %d]", k, SMILESS_MAX_INSTANCES);
    if (a->flags & SMILESS_FLAG_COST_CAP) {
        if (!(a->cost_cap >= 0.0)) return fail(ctx, SMILESS_EINVAL, "cost_cap must be >= 0 (not NaN)");
        if (a->flags & SMILESS_FLAG_NO_PRUNE) return fail(ctx, SMILESS_EINVAL, "FLAG_COST_CAP requires prune mode");
    }
    return SMILESS_OK;
}

std::string fmt_ll(long long v) { return std::to_string(v); }

// Choose the int32 chunk length K (or the int64 path): every relative value of a candidate
// still within the SLA must fit in int32.
struct RangePlan {
    bool time64;
    int K;
    i64 d_cap;
};

int inst_prologue(const smiless_ctx *ctx, const smiless_plan_args *a);
int inst_max(const smiless_ctx *ctx, const smiless_plan_args *a);

RangePlan range_plan(const smiless_ctx *ctx, const smiless_plan_args *a) {
    i64 wmax = a->windows_us[a->n_windows - 1];
    if (a->row_windows_us) {
        wmax = 0;
        for (int r = 0; r < ctx->sumM; ++r) wmax = std::max<i64>(wmax, a->row_windows_us[r]);
    }
    const i64 sla = a->sla_us;
    const i64 d_cap = sla + wmax + ctx->Tmax + 1;
    RangePlan rp{true, 64, d_cap};
    if (a->flags & SMILESS_FLAG_FORCE_INT64) return rp;
    const i64 LIM = 0x7fffffffll;
    // scale-out: the rings reach n_max - 1 requests back inside a frame, and the prologue
    // (j = 1 .. P) must lie in chunk 0 (K >= P)
    const i64 ring_span = (i64)(inst_max(ctx, a) - 1) * d_cap;
    const int P = inst_prologue(ctx, a);
    // SMILESS_FORCE_K (testing): use this chunk length if the int32 range rule holds for it
    // (else the int64 path), so the shorter-chunk variants are exercised on ordinary inputs
    if (const char *fk = getenv("SMILESS_FORCE_K")) {
        const int K = atoi(fk);
        if (K == 64 || K == 32 || K == 16 || K == 8 || K == 4) {
            const i64 bound = (i64)K * d_cap + sla + (i64)ctx->N * (ctx->Tmax + ctx->Imax) + wmax + ctx->Tmax +
                              (i64)K * ctx->Imax + ring_span;
            if (K >= P && bound < LIM && (i64)K * wmax < LIM) return RangePlan{false, K, d_cap};
            return rp;
        }
    }
    for (int K : {64, 32, 16, 8, 4}) {
        const i64 bound = (i64)K * d_cap + sla + (i64)ctx->N * (ctx->Tmax + ctx->Imax) + wmax + ctx->Tmax +
                          (i64)K * ctx->Imax + ring_span;
        if (K >= P && bound < LIM && (i64)K * wmax < LIM) return RangePlan{false, K, d_cap};
    }
    return rp;
}

// ------------------------------------------------------------------------------------
// NVRTC specialisation
// ------------------------------------------------------------------------------------
// Configs of the last function carried per lane (a unit = G x W candidates): as many as keep
// G * W <= 16 variants (registers) and divide M_{N-1}.  SMILESS_G overrides (tuning).
// Scale-out plans (NEXT-4, reading G26): a->instances[k] round-robin instances of function k.
int inst_of(const smiless_plan_args *a, int k) { return a->instances ? a->instances[k] : 1; }
int inst_max(const smiless_ctx *ctx, const smiless_plan_args *a) {
    int m = 1;
    for (int k = 0; k < ctx->N; ++k) m = std::max(m, inst_of(a, k));
    return m;
}
bool inst_mode(const smiless_ctx *ctx, const smiless_plan_args *a) { return inst_max(ctx, a) > 1; }
// the virtual sink (DESIGN.md section 5 item 13) is needed only when the LAST function scales
// out: otherwise its window variants keep sink sharing and the memoised throughput path, and
// only the upstream functions carry instance rings
// A scaled-out last function keeps its window variants with instance rings (evaluator.cuh
// variants_step_ring: sink sharing and the memoised path stay; C5 slice 2.9e7 -> 2.85e8
// candidates/s); SMILESS_LRING=0 uses the virtual sink instead (both are tested)
bool lring_on() {
    const char *e = getenv("SMILESS_LRING");
    return !e || atoi(e) != 0;
}
bool virt_sink(const smiless_ctx *ctx, const smiless_plan_args *a) { return inst_of(a, ctx->N - 1) > 1 && !lring_on(); }
// prologue steps j = 1 .. P of a scale-out plan (the first request of instances 2 .. n_k), a
// multiple of 4 so that the main loop keeps its 16-byte aligned offset loads
int inst_prologue(const smiless_ctx *ctx, const smiless_plan_args *a) {
    const int m = inst_max(ctx, a);
    return m > 1 ? ((m - 1 + 3) & ~3) : 0;
}

int configs_per_lane(const smiless_ctx *ctx, const smiless_plan_args *a) {
    if (virt_sink(ctx, a)) return 1;                 // last kernel function = the virtual sink (M = 1)
    const int M = ctx->M[ctx->N - 1], W = a->n_windows;
    int G = 1;
    const char *env = getenv("SMILESS_G");
    // per-row windows carry a run-time window and Te per variant: fewer variants fit in registers
    const int want = env ? std::max(1, atoi(env)) : (a->row_windows_us ? 8 : std::max(1, 16 / W));
    for (int g = 1; g <= want; ++g)
        if (M % g == 0 && g * W <= 32) G = g;
    return G;
}

// candidates per evaluator unit (lane): G configs x W windows of the last function; 1 for a
// scale-out plan, whose last kernel function is the virtual sink (one variant)
u64 unit_cands(const smiless_ctx *ctx, const smiless_plan_args *a) {
    return virt_sink(ctx, a) ? 1 : (u64)a->n_windows * (u64)configs_per_lane(ctx, a);
}
// window variants of the last kernel function
int variant_windows(const smiless_ctx *ctx, const smiless_plan_args *a) {
    return virt_sink(ctx, a) ? 1 : a->n_windows;
}

// The DAG the evaluator kernels are specialised for.  Normally the application DAG.  For a
// scale-out plan one virtual function V is appended: it joins every real sink, has one
// configuration (I = T = 0, U = 0: the spare zero table row), keep-alive, one instance, and its
// digit has radix 1 (the candidate index is unchanged).  Every real function is then an
// "upstream" function of the kernel and can carry an instance ring; V is the kernel's last
// function (sink sharing with one variant).  Cost: + U_V * E_V = + 0.0 (bit-exact).  Latency:
// D_V,j = max_{i <= j} x_i (running max, I = 0), so max_j (D_V,j - r_j) = max_j L_j exactly
// (r non-decreasing), which is all the SLA verdict and the pruning use.
struct KDag {
    int N = 0;
    bool virt = false;
    std::vector<std::vector<int>> preds;
    std::vector<int> M, row0, inst;
    u64 sink = 0;
};

KDag kernel_dag(const smiless_ctx *ctx, const smiless_plan_args *a) {
    KDag d;
    d.virt = virt_sink(ctx, a);
    d.N = ctx->N + (d.virt ? 1 : 0);
    d.preds.resize(d.N);
    d.M.resize(d.N);
    d.row0.resize(d.N);
    d.inst.resize(d.N, 1);
    for (int k = 0; k < ctx->N; ++k) {
        for (int e = ctx->pred_ptr[k]; e < ctx->pred_ptr[k + 1]; ++e) d.preds[k].push_back(ctx->pred_idx[e]);
        d.M[k] = ctx->M[k];
        d.row0[k] = ctx->row0[k];
        d.inst[k] = inst_of(a, k);
    }
    if (d.virt) {
        const int v = ctx->N;
        for (int k = 0; k < ctx->N; ++k)
            if ((ctx->sinkmask >> k) & 1ull) d.preds[v].push_back(k);
        d.M[v] = 1;
        d.row0[v] = ctx->sumM;
        d.sink = 1ull << v;
    } else {
        d.sink = ctx->sinkmask;
    }
    return d;
}

// Branch-and-bound depth D (functions 0..D-1 assigned per prefix, D..N-1 relaxed), or 0 for
// no pre-pass: prune mode, a large space, and a subtree of >= 4096 candidates per prefix.
// SMILESS_BB_DEPTH overrides (0 disables).
int bb_depth(const smiless_ctx *ctx, const smiless_plan_args *a) {
    if (a->flags & SMILESS_FLAG_NO_PRUNE) return 0;
    const int N = ctx->N, W = a->n_windows, nf = a->n_fixed;
    const char *env = getenv("SMILESS_BB_DEPTH");
    if (env) {
        const int d = atoi(env);
        return (d > nf && d <= N - 1) ? d : 0;
    }
    u64 space = 1;
    for (int k = nf; k < N; ++k) space *= (u64)ctx->M[k] * (u64)W;
    if (N < 3 || space < ((u64)1 << 26)) return 0;
    int best = 0;
    unsigned __int128 sub = (u64)ctx->M[N - 1] * (u64)W;
    for (int d = N - 2; d > nf; --d) {
        sub *= (u64)ctx->M[d] * (u64)W;                  // candidates per prefix of depth d
        if (sub >= 4096) { best = d; break; }
    }
    return best;
}

// Shallow B&B level (two-level scheme): the deepest depth < D with at most 2^22 prefixes (2^16
// for a sub-plan with pinned digits: C5's 128 function-0 digits are mostly pruned at this level,
// and a 2^21-prefix level took 0.13 ms per digit against ~0.02 ms for 2^14; C5 44 -> 39 ms,
// C5s 35 -> 30 ms, profiles/r02n_bb3.md), if the deep level has more than 2^24 prefixes (else 0:
// single level).  SMILESS_BB_DEPTH_A overrides.
int bb_depth_a(const smiless_ctx *ctx, const smiless_plan_args *a, int D) {
    if (D <= 0) return 0;
    const int nf = a->n_fixed, W = a->n_windows;
    const char *env = getenv("SMILESS_BB_DEPTH_A");
    if (env) {
        const int d = atoi(env);
        return (d > nf && d < D) ? d : 0;
    }
    unsigned __int128 prefD = 1;
    for (int k = nf; k < D; ++k) prefD *= (u64)ctx->M[k] * (u64)W;
    if (prefD <= ((unsigned __int128)1 << 24)) return 0;
    int best = 0;
    unsigned __int128 pref = 1;
    const unsigned __int128 cap = (unsigned __int128)1 << (nf > 0 ? 16 : 22);
    for (int d = nf + 1; d < D; ++d) {
        pref *= (u64)ctx->M[d - 1] * (u64)W;
        if (pref <= cap) best = d;
    }
    return best;
}

// Middle B&B level (three-level scheme): when every shallow survivor has more than 2^20 deep
// children, a level at DM = DA + ceil((D - DA) / 2) prunes them first, so the deep level only
// enumerates the children of middle survivors (C5: 2^28 deep children per shallow survivor
// become 2 x 2^14; C5 437 -> 57 ms, C5s 232 -> 51 ms; C3's 2^19.8 measured 12 -> 14 ms with it,
// so it stays at two levels; profiles/r02n_bb3.md).  0: none.  SMILESS_BB_DEPTH_M overrides.
int bb_depth_m(const smiless_ctx *ctx, const smiless_plan_args *a, int D, int DA) {
    if (D <= 0 || DA <= 0) return 0;
    const char *env = getenv("SMILESS_BB_DEPTH_M");
    if (env) {
        const int d = atoi(env);
        return (d > DA && d < D) ? d : 0;
    }
    if (D - DA < 2) return 0;
    unsigned __int128 r = 1;
    for (int k = DA; k < D; ++k) r *= (u64)ctx->M[k] * (u64)a->n_windows;
    if (r <= ((unsigned __int128)1 << 20)) return 0;
    return DA + (D - DA + 1) / 2;
}

u64 cands_per_prefix(const smiless_ctx *ctx, const smiless_plan_args *a, int d) {
    u64 s = 1;
    for (int k = d; k < ctx->N; ++k) s *= (u64)ctx->M[k] * (u64)a->n_windows;
    return s;
}

enum { FAM_PLAN = 1, FAM_BOUND = 2, FAM_MEMO = 4, FAM_ALL = 7 };   // kernel families of a module

// Throughput mode with prefix memoisation: walk every unit without the sum-of-u accumulators
// and re-walk only the units holding a feasible candidate to finish their costs (DESIGN.md
// section 5 item 12; +3 % candidates/s on the C2 slice).  On by default; SMILESS_SPLITCOST=0
// walks every unit with the accumulators in one pass.
bool split_cost() {
    const char *e = getenv("SMILESS_SPLITCOST");
    return !e || atoi(e) != 0;
}

// Fused memoisation (evaluator.cuh smiless_fused_kernel): one persistent kernel whose producer
// warp walks the upstream functions of a tile of prefixes into a shared-memory ring that its
// consumer warps read, so the x stream never leaves the SM.  Needs the int32 path, a last
// function that is not scaled out, and a tile of 1..32 prefixes.  SMILESS_FUSED=0: two kernels.
constexpr int kFusedSteps = 64;                      // mirrors SM_FPS
int fused_slots() {                                  // ring depth (SM_FSLOTS)
    const char *e = getenv("SMILESS_FSLOTS");
    const int v = e ? atoi(e) : 4;
    return (v >= 2 && v <= 8) ? v : 4;
}
int fused_min_blocks() {                             // min CTAs/SM of the fused kernel (SM_FMINB)
    const char *e = getenv("SMILESS_FMINB");
    const int v = e ? atoi(e) : 1;
    return (v >= 1 && v <= 4) ? v : 1;
}
// Default shape: one 640-thread CTA per SM, 16 consumer warps and 4 producer warps (16 lanes
// each), so each SM sub-partition runs 4 consumers and 1 producer (profiles/r02l_memo_batch.md:
// with the producers on one SMSP its issue rate fell to 51 %)
int fused_producers() {                              // producer warps per CTA (SM_FPW)
    const char *e = getenv("SMILESS_FPW");
    const int v = e ? atoi(e) : 4;
    return (v >= 1 && v <= 8) ? v : 4;
}
int fused_threads() {                                // CTA size (SM_FTHREADS)
    const char *e = getenv("SMILESS_FTHREADS");
    const int v = e ? atoi(e) : 640;
    return (v >= 64 && v <= 1024 && v % 32 == 0) ? v : 640;
}
int fused_tile(const smiless_ctx *ctx, const smiless_plan_args *a) {
    return (fused_threads() / 32 - fused_producers()) * 32 / (ctx->M[ctx->N - 1] / configs_per_lane(ctx, a));
}
bool fused_on(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp) {
    const char *e = getenv("SMILESS_FUSED");
    if (e && atoi(e) == 0) return false;
    if (rp.time64 || inst_of(a, ctx->N - 1) > 1) return false;
    const int tp = fused_tile(ctx, a), fpw = fused_producers();
    return tp >= 1 && (tp + fpw - 1) / fpw <= 32 && 32 * fpw <= kThreads;
}
size_t smem_fused(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, i64 n_off) {
    const size_t padI = (size_t)((ctx->sumM + 3) & ~3), padU = (size_t)((ctx->sumM + 1) & ~1);
    const size_t fc32 = (size_t)(fused_threads() / 32 - fused_producers()) * 32;
    (void)rp;
    return 3 * padI * 4 + padU * 8 + 4 * (size_t)n_off + (split_cost() ? 0 : 8 * (size_t)unit_cands(ctx, a) * fc32) +
           4 * (size_t)fused_slots() * kFusedSteps * (size_t)fused_tile(ctx, a) +
           ((4 * (size_t)ctx->N * kThreads + 15) & ~(size_t)15);
}

// static cost-bound terms of every (row, window) staged in shared memory when small
bool bound_lb_table(const smiless_ctx *ctx, int W) { return (size_t)ctx->sumM * (size_t)W <= 8192; }

std::string dag_spec_source(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, bool off_smem,
                            int minb, int families) {
    const KDag kd = kernel_dag(ctx, a);
    const int N = kd.N, W = a->n_windows, NU = N - 1, nf = a->n_fixed;
    const int G = configs_per_lane(ctx, a);
    const int VW = variant_windows(ctx, a);
    const int P = inst_prologue(ctx, a);
    const char *un_env = getenv("SMILESS_UNROLL");
    const int unroll = (un_env && atoi(un_env) == 2) ? 2 : 4;
    // instance rings: function k keeps its n_k - 1 older completions in RG[rg0[k] ..]
    std::vector<int> rg0(N, 0);
    int n_rg = 0;
    for (int k = 0; k < N; ++k) {
        rg0[k] = n_rg;
        n_rg += kd.inst[k] - 1;
    }
    std::ostringstream s;
    s << "// generated by host.cpp:dag_spec_source -- DAG-specialised prefix of evaluator.cuh\n";
    s << "#define SM_N " << N << "\n#define SM_NU " << NU << "\n#define SM_NU_ALLOC " << std::max(NU, 1) << "\n";
    s << "#define SM_W " << W << "\n#define SM_NFIXED " << nf << "\n#define SM_NFIXED_ALLOC " << SMILESS_MAX_FUNCS
      << "\n";
    s << "#define SM_K " << rp.K << "\n#define SM_TIME64 " << (rp.time64 ? 1 : 0) << "\n";
    s << "#define SM_OFF_SMEM " << (off_smem ? 1 : 0) << "\n#define SM_THREADS " << kThreads
      << "\n#define SM_MINB " << minb << "\n";
    // window variants of the last kernel function: the grid, or the virtual sink's keep-alive
    s << "#define SM_VW " << VW << "\n";
    s << "#define SM_W0_ZERO " << (kd.virt || (!a->row_windows_us && a->windows_us[0] == 0) ? 1 : 0) << "\n";
    s << "#define SM_G " << G << "\n#define SM_UNROLL " << unroll << "\n";
    s << "#define SM_UPP " << (kd.M[N - 1] / G) << "\n";   // units (config groups) per upstream prefix
    s << "#define SM_VTHREADS " << vthreads_per_cta() << "\n#define SM_VMINB " << vmin_blocks() << "\n";
    s << "#define SM_BUILD_PLAN " << ((families & FAM_PLAN) ? 1 : 0) << "\n#define SM_BUILD_BOUND "
      << ((families & FAM_BOUND) ? 1 : 0) << "\n#define SM_BUILD_MEMO " << ((families & FAM_MEMO) ? 1 : 0) << "\n";
    const char *ck_env = getenv("SMILESS_CHECK");     // SLA early-exit check period (steps)
    const int check = std::max(unroll, ck_env ? atoi(ck_env) : 16);
    s << "#define SM_CHECK " << check << "\n";
    const int D = bb_depth(ctx, a);
    const int DA = bb_depth_a(ctx, a, D);
    s << "#define SM_D " << (D > 0 ? D : N - 1) << "\n#define SM_DA " << (DA > 0 ? DA : (D > 0 ? D : N - 1))
      << "\n#define SM_DM " << bb_depth_m(ctx, a, D, DA) << "\n#define SMILESS_MAXF " << SMILESS_MAX_FUNCS << "\n";
    s << "#define SM_NSLA " << ctx->nsla << "\n";
    s << "#define SM_ROWWIN " << (a->row_windows_us ? 1 : 0) << "\n";
    s << "#define SM_LBT " << (bound_lb_table(ctx, W) ? 1 : 0) << "\n";
    s << "#define SM_XPF " << xpf_groups() << "\n";
    s << "#define SM_SPLITCOST " << (split_cost() ? 1 : 0) << "\n";
    s << "#define SM_FUSED " << (((families & FAM_MEMO) && fused_on(ctx, a, rp)) ? 1 : 0) << "\n#define SM_FSLOTS "
      << fused_slots() << "\n#define SM_FMINB " << fused_min_blocks() << "\n#define SM_FPW " << fused_producers()
      << "\n#define SM_FTHREADS " << fused_threads() << "\n";
    // window variants of the memoised kernel walked in the positive-time form (evaluator.cuh
    // variants_step FM: ALU busy mask + full-rate IMAD instead of the quarter-rate IMAD.HI)
    // default: every window variant (measured: 3.45e8 -> 3.81e8 candidates/s on the C2 slice,
    // profiles/r02_sweep_fmask.md); the keep-alive variant needs no mask either way
    const char *fm_env = getenv("SMILESS_FMASK");
    s << "#define SM_FMASK " << (fm_env ? strtoul(fm_env, nullptr, 0) : 0xfffffffful) << "u\n";
    // scale-out (NEXT-4): any instance count > 1, the prologue length, the ring size
    s << "#define SM_INST " << (inst_mode(ctx, a) ? 1 : 0) << "\n#define SM_VIRT " << (kd.virt ? 1 : 0)
      << "\n#define SM_PRO " << P << "\n#define SM_RG_ALLOC "
      << std::max(n_rg, 1) << "\n";
    s << "#define SM_NL " << (kd.virt ? 1 : kd.inst[N - 1]) << "\n";   // instances of the variants' function
    s << "#define SM_NINST(k) (";
    for (int k = 0; k < N; ++k) s << "(k)==" << k << "?" << kd.inst[k] << ":";
    s << "1)\n";
    s << "#define SM_ROWINST(r) (";                      // instances of the function owning table row r
    for (int k = 0; k < N; ++k) s << "(r)<" << kd.row0[k] + kd.M[k] << "?" << kd.inst[k] << ":";
    s << "1)\n";
    // compile-time window grid (immediates) and a constant-bank copy for runtime indices
    s << "#define SM_WIN(v) (";
    for (int v = 0; v < W; ++v) s << "(v)==" << v << "?" << a->windows_us[v] << ":";
    s << "0)\n";
    // windows of the last kernel function's variants (the virtual sink: keep-alive)
    s << "#define SM_VWIN(v) " << (kd.virt ? "0" : "SM_WIN(v)") << "\n";
    s << "__constant__ int c_win[" << W << "] = {";
    for (int v = 0; v < W; ++v) s << (v ? "," : "") << a->windows_us[v];
    s << "};\n#define SM_WINV(i) c_win[(i)]\n";
    s << "#define SM_ROW0(k) (";
    for (int k = 0; k < N; ++k) s << "(k)==" << k << "?" << kd.row0[k] << ":";
    s << "0)\n";
    s << "#define SM_MK(k) (";
    for (int k = 0; k < N; ++k) s << "(k)==" << k << "?" << kd.M[k] << ":";
    s << "0)\n";
    s << R"(
typedef long long i64;
typedef unsigned long long u64;
#if SM_TIME64
typedef long long tm_t;
#else
typedef int tm_t;
#endif
static __device__ __forceinline__ void fstep(tm_t &NF, tm_t &SU, tm_t g, tm_t NI, tm_t Te, tm_t w);
static __device__ __forceinline__ tm_t vminz(tm_t a, tm_t b, tm_t z);
static __device__ __forceinline__ tm_t vaddmin(tm_t a, tm_t b, tm_t c);
static __device__ __forceinline__ tm_t opaque_add(tm_t a, tm_t b);
static __device__ __forceinline__ tm_t opaque_sub(tm_t a, tm_t b);
static __device__ __forceinline__ tm_t vaddmax(tm_t a, tm_t b, tm_t c);
static __device__ __forceinline__ tm_t vmax(tm_t a, tm_t b);
)";
    // ---- decode: unit u -> digits (last kernel function: config group only) ---------------
    s << "static __device__ __forceinline__ void dag_decode(u64 u, int (&dig)[SM_N], const int *fixed) {\n";
    if (nf <= N - 1) {
        const int groups = kd.M[N - 1] / G;   // config groups of the last function
        s << "  dig[" << N - 1 << "] = (int)(u % " << groups << "ull); u /= " << groups << "ull;\n";
        for (int k = N - 2; k >= nf; --k) {
            const u64 radix = (u64)kd.M[k] * (u64)W;
            s << "  dig[" << k << "] = (int)(u % " << radix << "ull); u /= " << radix << "ull;\n";
        }
    }
    for (int k = 0; k < nf; ++k) s << "  dig[" << k << "] = fixed[" << k << "];\n";
    s << "  (void)u; (void)fixed;\n}\n";

    // ---- input expressions, negated time (NF = -F) ---------------------------------------
    // min over predecessors of NF (= -(max over predecessors of F): the AND-join).
    // vminz blocks VIMNMX3 formation (ptxas erratum); nothing below negates a min/max input.
    auto nf_min = [&](int k) {
        const auto &pr = kd.preds[k];
        std::string e = "NF[" + std::to_string(pr[0]) + "]";
        for (size_t i = 1; i < pr.size(); ++i) e = "vminz(" + e + ", NF[" + std::to_string(pr[i]) + "], z)";
        return e;
    };
    auto is_src = [&](int k) { return kd.preds[k].empty(); };
    auto ks = [](int k) { return std::to_string(k); };
    // ---- j = 0: start = x; nx = -x is stored (st0); scale-out functions start EF = D_0 - r_0 --
    s << "template <int A> static __device__ __forceinline__ void dag_first(tm_t (&NF)[A], const tm_t (&NI)[A], "
         "tm_t *st0, int tid, tm_t &nxl, tm_t &nlu, const tm_t z, i64 (&EF)[A]) {\n";
    for (int k = 0; k < N - 1; ++k) {
        s << "  { const tm_t nx = " << (is_src(k) ? std::string("(tm_t)0") : nf_min(k)) << "; st0[" << k
          << " * SM_THREADS + tid] = nx; NF[" << k << "] = NI[" << k << "] + nx; }\n";
        if (kd.inst[k] > 1) s << "  EF[" << k << "] = -(i64)NF[" << k << "];\n";
    }
    s << "  nxl = " << (is_src(N - 1) ? std::string("(tm_t)0") : nf_min(N - 1)) << ";\n";
    for (int k = 0; k < N - 1; ++k)
        if ((kd.sink >> k) & 1ull) s << "  nlu = vminz(nlu, NF[" << k << "], z);\n";
    s << "  (void)NF; (void)NI; (void)st0; (void)tid; (void)nlu; (void)z; (void)EF;\n}\n";
    // ---- j >= 1: g = x - f = x + NF; returns x of the last function ----------------------
    // JJ = 0: steady state; JJ >= 1: prologue step j = JJ of a scale-out plan, where a function
    // with JJ < n_k serves the first request of instance JJ (pre-warmed, G5: start = x, no u).
    // Instance rings: f = RG[rg0] (completion n_k requests back), shifted each step; NF[k] is
    // always the newest completion (what the joins and sinks read).
    s << "template <int JJ, int A, int R> static __device__ __forceinline__ tm_t dag_step(tm_t (&NF)[A], tm_t (&RG)[R], "
         "tm_t (&SU)[A], const tm_t (&NI)[A], const tm_t (&Te)[A], const tm_t (&Wn)[A], const tm_t o, const tm_t z, "
         "i64 (&EF)[A]) {\n";
    for (int k = 0; k < N - 1; ++k) {
        const int n = kd.inst[k];
        if (n == 1) {
            const std::string g = is_src(k) ? "o + NF[" + ks(k) + "]" : "NF[" + ks(k) + "] - " + nf_min(k);
            s << "  fstep(NF[" << k << "], SU[" << k << "], " << g << ", NI[" << k << "], Te[" << k << "], Wn[" << k
              << "]);\n";
            continue;
        }
        const std::string nx = is_src(k) ? std::string("opaque_sub(z, o)") : nf_min(k);   // -x
        s << "  {\n";
        s << "    tm_t nf = RG[" << rg0[k] << "];\n";
        for (int r = 0; r + 1 < n - 1; ++r) s << "    RG[" << rg0[k] + r << "] = RG[" << rg0[k] + r + 1 << "];\n";
        s << "    RG[" << rg0[k] + n - 2 << "] = NF[" << k << "];\n";
        s << "    if (JJ != 0 && JJ < " << n << ") {\n";
        s << "      NF[" << k << "] = NI[" << k << "] + " << nx << ";\n";
        s << "      EF[" << k << "] += -(i64)NF[" << k << "] - (i64)o;\n";
        s << "    } else {\n";
        const std::string g = is_src(k) ? std::string("o + nf") : "nf - " + nf_min(k);
        s << "      fstep(nf, SU[" << k << "], " << g << ", NI[" << k << "], Te[" << k << "], Wn[" << k << "]);\n";
        s << "      NF[" << k << "] = nf;\n";
        s << "    }\n  }\n";
    }
    s << "  (void)NF; (void)RG; (void)SU; (void)NI; (void)Te; (void)Wn; (void)o; (void)z; (void)EF;\n";
    s << "  return " << (is_src(N - 1) ? std::string("o") : "opaque_sub(z, " + nf_min(N - 1) + ")") << ";\n}\n";
    // ---- scale-out billing: sum_{i < n_eff} (D_{J-1-i} - r_{J-1-i}) from the final ring -------
    s << "template <int A, int R> static __device__ __forceinline__ i64 dag_elast(const int k, const tm_t (&NF)[A], "
         "const tm_t (&RG)[R], const i64 *otail, const i64 J) {\n  i64 e = 0;\n";
    for (int k = 0; k < N - 1; ++k) {
        const int n = kd.inst[k];
        if (n == 1) continue;
        s << "  if (k == " << k << ") {\n    e = -(i64)NF[" << k << "] - otail[0];\n";
        for (int i = 1; i < n; ++i)
            s << "    if (J > " << i << ") e += -(i64)RG[" << rg0[k] + n - 1 - i << "] - otail[" << i << "];\n";
        s << "  }\n";
    }
    s << "  (void)NF; (void)RG; (void)otail; (void)J; (void)k;\n  return e;\n}\n";
    // ---- rebase of the instance rings (F -= sh  <=>  NF += sh) ---------------------------
    s << "template <int R> static __device__ __forceinline__ void dag_ring_rebase(tm_t (&RG)[R], const tm_t sh) {\n";
    for (int r = 0; r < n_rg; ++r) s << "  RG[" << r << "] += sh;\n";
    s << "  (void)RG; (void)sh;\n}\n";
    // ---- upstream sinks' latency: nlu = min_j (NF_k + o_j) = -max_j L_j -------------------
    s << "template <int A> static __device__ __forceinline__ void dag_sinks(const tm_t (&NF)[A], const tm_t o, tm_t "
         "&nlu) {\n";
    for (int k = 0; k < N - 1; ++k)
        if ((kd.sink >> k) & 1ull) s << "  nlu = vaddmin(NF[" << k << "], o, nlu);\n";
    s << "  (void)NF; (void)o; (void)nlu;\n}\n";
    // ---- B&B pre-pass (smiless_bound_kernel): prefix decode, relaxed first/step ---------------
    {
        s << "template <int DD> static __device__ __forceinline__ void dag_bdecode(u64 u, int (&dig)[SM_N], "
             "const int *fixed) {\n";
        for (int k = 0; k < N; ++k) s << "  dig[" << k << "] = 0;\n";
        for (int k = N - 1; k >= nf; --k) {
            const u64 radix = (u64)kd.M[k] * (u64)W;
            s << "  if (" << k << " < DD) { dig[" << k << "] = (int)(u % " << radix << "ull); u /= " << radix
              << "ull; }\n";
        }
        for (int k = 0; k < nf; ++k) s << "  dig[" << k << "] = fixed[" << k << "];\n";
        s << "  (void)u; (void)fixed;\n}\n";
        s << "template <int A> static __device__ __forceinline__ void dag_bfirst(tm_t (&NF)[A], const tm_t (&NI)[A], "
             "tm_t &nl, const tm_t z) {\n";
        for (int k = 0; k < N; ++k)
            s << "  NF[" << k << "] = NI[" << k << "] + " << (is_src(k) ? std::string("(tm_t)0") : nf_min(k)) << ";\n";
        for (int k = 0; k < N; ++k)
            if ((kd.sink >> k) & 1ull) s << "  nl = vminz(nl, NF[" << k << "], z);\n";
        s << "  (void)z;\n}\n";
        // Lower bounds of every done time.  An assigned function (k < DD) has exact inputs (all its
        // predecessors are assigned) and runs model M exactly, with its instance ring.  A relaxed
        // function (k >= DD) runs keep-alive on its smallest exec time: max(x', D'_{j-n}) + I_min
        // (a ring of n_k - 1 older bounds for n_k > 1; the first request of an instance x' + I_min)
        // -- in every branch of model M start >= max(x, D_{j-n}), and that bound is monotone in its
        // lower-bounded inputs.
        s << "template <int DD, int JJ, int A, int R> static __device__ __forceinline__ void dag_bstep(tm_t (&NF)[A], "
             "tm_t (&RG)[R], const tm_t (&NI)[A], const tm_t (&Te)[A], const tm_t (&Wn)[A], const tm_t o, tm_t &nl, "
             "const tm_t z) {\n  tm_t su = 0;\n";
        for (int k = 0; k < N; ++k) {
            const int n = kd.inst[k];
            const std::string nx = is_src(k) ? std::string("opaque_sub(z, o)") : nf_min(k);
            if (n == 1) {
                const std::string g = is_src(k) ? "o + NF[" + ks(k) + "]" : "NF[" + ks(k) + "] - " + nf_min(k);
                s << "  if (" << k << " < DD) fstep(NF[" << k << "], su, " << g << ", NI[" << k << "], Te[" << k
                  << "], Wn[" << k << "]);\n  else { const tm_t g = " << g << "; NF[" << k << "] = NF[" << k
                  << "] + NI[" << k << "] - vmax(g, (tm_t)0); }\n";
                continue;
            }
            const std::string g = is_src(k) ? std::string("o + nf") : "nf - " + nf_min(k);
            s << "  {\n    tm_t nf = RG[" << rg0[k] << "];\n";
            for (int r = 0; r + 1 < n - 1; ++r) s << "    RG[" << rg0[k] + r << "] = RG[" << rg0[k] + r + 1 << "];\n";
            s << "    RG[" << rg0[k] + n - 2 << "] = NF[" << k << "];\n";
            s << "    if (JJ != 0 && JJ < " << n << ") NF[" << k << "] = NI[" << k << "] + " << nx << ";\n";
            s << "    else if (" << k << " < DD) { fstep(nf, su, " << g << ", NI[" << k << "], Te[" << k << "], Wn[" << k
              << "]); NF[" << k << "] = nf; }\n";
            s << "    else { const tm_t g = " << g << "; NF[" << k << "] = nf + NI[" << k << "] - vmax(g, (tm_t)0); }\n";
            s << "  }\n";
        }
        for (int k = 0; k < N; ++k)
            if ((kd.sink >> k) & 1ull) s << "  nl = vaddmin(NF[" << k << "], o, nl);\n";
        s << "  (void)su; (void)Te; (void)Wn; (void)z;\n}\n";
    }
    return s.str();
}

std::string full_source(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, bool off_smem,
                        int minb, int families = FAM_ALL) {
    if (virt_sink(ctx, a)) families &= ~FAM_MEMO;       // a scaled-out last function: no memo path
    return dag_spec_source(ctx, a, rp, off_smem, minb, families) + "\n" + smiless_evaluator_src;
}

// shared-memory bytes of the memo kernels / bound kernel (host-side, to pick a path before compiling)
size_t smem_memo_up(const smiless_ctx *ctx, const RangePlan &rp, i64 n_off) {
    const size_t padI = (size_t)((ctx->sumM + 3) & ~3), padU = (size_t)((ctx->sumM + 1) & ~1);
    const size_t tsz = rp.time64 ? 8 : 4;
    return 3 * padI * 4 + padU * 8 + tsz * (size_t)n_off + 8ull * (size_t)std::max(ctx->N - 1, 1) * kThreads +
           ((tsz * (size_t)ctx->N * kThreads + 15) & ~(size_t)15);
}
size_t smem_memo_var(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, i64 n_off);
// table rows the plan / bound kernels stage: a scale-out plan adds the virtual sink's zero row
int kernel_rows(const smiless_ctx *ctx, const smiless_plan_args *a) { return ctx->sumM + (virt_sink(ctx, a) ? 1 : 0); }
int kernel_funcs(const smiless_ctx *ctx, const smiless_plan_args *a) { return ctx->N + (virt_sink(ctx, a) ? 1 : 0); }

size_t smem_bound_bytes(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, i64 n_off) {
    const int rows = kernel_rows(ctx, a);
    const size_t padI = (size_t)((rows + 3) & ~3);
    const size_t lbt = bound_lb_table(ctx, a->n_windows) ? 8 * (size_t)((rows * a->n_windows + 1) & ~1) : 0;
    return 3 * padI * 4 + 8 * (size_t)((rows + 1) & ~1) + lbt + (rp.time64 ? 8 : 4) * (size_t)n_off;
}

int nvrtc_compile(smiless_ctx *ctx, const std::string &src, std::vector<char> &cubin, std::string &log) {
    NvrtcApi &nv = nvrtc();
    if (!nv.ok) return fail(ctx, SMILESS_EJIT, "NVRTC unavailable: %s", nv.why.c_str());
    nvrtcProgram prog;
    nvrtcResult r = nv.create(&prog, src.c_str(), "smiless_evaluator.cu", 0, nullptr, nullptr);
    if (r != NVRTC_SUCCESS) return fail(ctx, SMILESS_EJIT, "nvrtcCreateProgram: %s", nv.err_str(r));
    const char *opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-default-device", "-lineinfo", "-fmad=false",
                          "--ptxas-options=-v"};
    r = nv.compile(prog, (int)(sizeof opts / sizeof *opts), opts);
    size_t ls = 0;
    nv.log_size(prog, &ls);
    log.assign(ls, '\0');
    if (ls) nv.get_log(prog, &log[0]);
    if (r != NVRTC_SUCCESS) {
        nv.destroy(&prog);
        return fail(ctx, SMILESS_EJIT, "NVRTC compile failed: %s\n%s", nv.err_str(r), log.c_str());
    }
    size_t cs = 0;
    nv.cubin_size(prog, &cs);
    cubin.resize(cs);
    nv.get_cubin(prog, cubin.data());
    nv.destroy(&prog);
    return SMILESS_OK;
}

size_t smem_bytes(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, i64 n_off, bool off_smem) {
    const int rows = kernel_rows(ctx, a), kn = kernel_funcs(ctx, a);
    const size_t padI = (size_t)((rows + 3) & ~3);
    const size_t padU = (size_t)((rows + 1) & ~1);
    const size_t tsz = rp.time64 ? 8 : 4;
    size_t b = 3 * padI * 4 + padU * 8;
    b += 8ull * (size_t)(kn - 1 + (int)unit_cands(ctx, a)) * kThreads;
    b += (tsz * (size_t)kn * kThreads + 15) & ~(size_t)15;
    if (off_smem) b += tsz * (size_t)n_off;
    return b;
}

size_t smem_memo_var(const smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, i64 n_off) {
    const size_t padI = (size_t)((ctx->sumM + 3) & ~3), padU = (size_t)((ctx->sumM + 1) & ~1);
    const size_t tsz = rp.time64 ? 8 : 4;
    return 3 * padI * 4 + padU * 8 + tsz * (size_t)n_off +
           8ull * (size_t)(a->n_windows * configs_per_lane(ctx, a)) * vthreads_per_cta();
}

// tuning knob: min CTAs/SM for __launch_bounds__ of the evaluator / variants kernels
int min_blocks() {
    const char *mb_env = getenv("SMILESS_MINB");
    return mb_env ? std::max(1, atoi(mb_env)) : 1;
}

int get_kernel(smiless_ctx *ctx, const smiless_plan_args *a, const RangePlan &rp, i64 n_off, int families,
               JitKernel **out) {
    // offsets in shared memory when they fit next to the per-thread accumulators
    const size_t max_smem = 227 * 1024;
    bool off_smem = smem_bytes(ctx, a, rp, n_off, true) <= max_smem;
    std::string src = full_source(ctx, a, rp, off_smem, min_blocks(), families);
    auto it = ctx->jit_cache.find(src);
    if (it == ctx->jit_cache.end()) {
        std::vector<char> cubin;
        std::string log;
        int rc = nvrtc_compile(ctx, src, cubin, log);
        if (rc) return rc;
        JitKernel jk;
        CUresult r = driver().moduleLoadData(&jk.mod, cubin.data());
        if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleLoadData");
        if (families & FAM_PLAN) {
            r = driver().moduleGetFunction(&jk.fn, jk.mod, "smiless_plan_kernel");
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction");
            jk.smem = smem_bytes(ctx, a, rp, n_off, off_smem);
            r = driver().funcSetAttribute(jk.fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)jk.smem);
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(smem)");
            driver().funcGetAttribute(&jk.regs, CU_FUNC_ATTRIBUTE_NUM_REGS, jk.fn);
            r = driver().occupancy(&jk.blocks_per_sm, jk.fn, kThreads, jk.smem);
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuOccupancyMaxActiveBlocksPerMultiprocessor");
            if (jk.blocks_per_sm < 1)
                return fail(ctx, SMILESS_ECUDA, "evaluator does not fit on an SM (smem %zu)", jk.smem);
        }
        if (families & FAM_BOUND) {
            r = driver().moduleGetFunction(&jk.fn_bound, jk.mod, "smiless_bound_kernel");
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(bound)");
            r = driver().moduleGetFunction(&jk.fn_bound_a, jk.mod, "smiless_bound_kernel_a");
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(bound_a)");
            const int D = bb_depth(ctx, a);
            if (bb_depth_m(ctx, a, D, bb_depth_a(ctx, a, D)) > 0) {
                r = driver().moduleGetFunction(&jk.fn_bound_m, jk.mod, "smiless_bound_kernel_m");
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(bound_m)");
            }
        }
        if (families & FAM_MEMO) {
            r = driver().moduleGetFunction(&jk.fn_up, jk.mod, "smiless_upstream_kernel");
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(upstream)");
            r = driver().moduleGetFunction(&jk.fn_var, jk.mod, "smiless_variants_kernel");
            if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(variants)");
            if (split_cost()) {
                r = driver().moduleGetFunction(&jk.fn_varc, jk.mod, "smiless_variants_cost_kernel");
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(variants cost)");
            }
        }
        if (families & FAM_MEMO) {
            const size_t padI = (size_t)((ctx->sumM + 3) & ~3), padU = (size_t)((ctx->sumM + 1) & ~1);
            const size_t tsz = rp.time64 ? 8 : 4;
            const size_t base = 3 * padI * 4 + padU * 8 + tsz * (size_t)n_off;
            jk.smem_up = base + 8ull * (size_t)std::max(ctx->N - 1, 1) * kThreads +
                         ((tsz * (size_t)ctx->N * kThreads + 15) & ~(size_t)15);
            jk.smem_var = base + 8ull * (size_t)(a->n_windows * configs_per_lane(ctx, a)) * vthreads_per_cta();
            if (jk.smem_up <= 227 * 1024 && jk.smem_var <= 227 * 1024) {
                r = driver().funcSetAttribute(jk.fn_up, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)jk.smem_up);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(upstream smem)");
                r = driver().funcSetAttribute(jk.fn_var, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                              (int)jk.smem_var);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(variants smem)");
                if (jk.fn_varc) {
                    r = driver().funcSetAttribute(jk.fn_varc, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                                  (int)jk.smem_var);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(variants cost smem)");
                }
                r = driver().occupancy(&jk.blocks_up, jk.fn_up, kThreads, jk.smem_up);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "occupancy(upstream)");
                r = driver().occupancy(&jk.blocks_var, jk.fn_var, vthreads_per_cta(), jk.smem_var);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "occupancy(variants)");
            }
            jk.smem_fused = smem_fused(ctx, a, rp, n_off);
            if (fused_on(ctx, a, rp) && jk.smem_fused <= 227 * 1024) {
                r = driver().moduleGetFunction(&jk.fn_fused, jk.mod, "smiless_fused_kernel");
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuModuleGetFunction(fused)");
                r = driver().funcSetAttribute(jk.fn_fused, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                              (int)jk.smem_fused);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(fused smem)");
                r = driver().occupancy(&jk.blocks_fused, jk.fn_fused, fused_threads(), jk.smem_fused);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "occupancy(fused)");
                if (jk.blocks_fused < 1) jk.fn_fused = nullptr;
            }
        }
        if (families & FAM_BOUND) {
            jk.smem_bound = smem_bound_bytes(ctx, a, rp, n_off);
            if (jk.smem_bound <= 227 * 1024) {
                r = driver().funcSetAttribute(jk.fn_bound, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                              (int)jk.smem_bound);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(bound smem)");
                r = driver().funcSetAttribute(jk.fn_bound_a, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                              (int)jk.smem_bound);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(bound_a smem)");
                if (jk.fn_bound_m) {
                    r = driver().funcSetAttribute(jk.fn_bound_m, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                                  (int)jk.smem_bound);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "cuFuncSetAttribute(bound_m smem)");
                }
                r = driver().occupancy(&jk.blocks_bound, jk.fn_bound, kThreads, jk.smem_bound);
                if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "occupancy(bound)");
            }
        }
        it = ctx->jit_cache.emplace(src, jk).first;
    }
    *out = &it->second;
    return SMILESS_OK;
}

void fill_exact_params(const smiless_ctx *ctx, const smiless_plan_args *a, const i64 *d_arr, ExactParams &ep) {
    memset(&ep, 0, sizeof ep);
    ep.tabI = ctx->dI.p;
    ep.tabT = ctx->dT.p;
    ep.tabU = ctx->dU.p;
    ep.arr = (const long long *)d_arr;
    ep.J = a->n_arrivals;
    ep.sla = a->sla_us;
    ep.N = ctx->N;
    ep.W = a->n_windows;
    ep.n_fixed = a->n_fixed;
    ep.sinkmask = (unsigned)ctx->sinkmask;
    ep.pred_ptr = ctx->dPtr.p;
    ep.pred_idx = ctx->dIdx.p;
    for (int k = 0; k < ctx->N; ++k) {
        ep.M[k] = ctx->M[k];
        ep.row0[k] = ctx->row0[k];
    }
    for (int v = 0; v < a->n_windows; ++v) ep.win[v] = a->windows_us[v];
    ep.rowwin = a->row_windows_us ? ctx->dW.p : nullptr;
    for (int k = 0; k < ctx->N; ++k) ep.inst[k] = inst_of(a, k);
    for (int k = 0; k < a->n_fixed; ++k) ep.fixed[k] = a->fixed_digits[k];
}

// Per-row windows of this call (row_windows_us) or zeros: the kernels always stage the table.
int stage_row_windows(smiless_ctx *ctx, const smiless_plan_args *a) {
    const size_t padI = (size_t)((ctx->sumM + 1 + 3) & ~3);
    std::vector<int> w(padI, 0);
    if (a->row_windows_us) std::copy(a->row_windows_us, a->row_windows_us + ctx->sumM, w.begin());
    if (ctx->dW.p && ctx->dW.n >= padI && w == ctx->hW && !ctx->tables_dirty) return SMILESS_OK;  // unchanged
    CK(ctx->dW.ensure(padI), "cudaMalloc row windows");
    CK(cudaMemcpyAsync(ctx->dW.p, w.data(), padI * sizeof(int), cudaMemcpyHostToDevice, ctx->stream), "H2D windows");
    ctx->h2d += padI * sizeof(int);
    ctx->hW.swap(w);
    return SMILESS_OK;
}

// Upload (host) or adopt (device) the arrival sequence; returns the device pointer.
int stage_arrivals(smiless_ctx *ctx, const smiless_plan_args *a, const i64 **d_arr) {
    if (a->flags & SMILESS_FLAG_ARRIVALS_ON_DEVICE) {
        *d_arr = (const i64 *)a->arrivals_us;
        return SMILESS_OK;
    }
    CK(ctx->dArr.ensure((size_t)a->n_arrivals), "cudaMalloc arrivals");
    ctx->h2d += (size_t)a->n_arrivals * sizeof(i64);
    CK(cudaMemcpyAsync(ctx->dArr.p, a->arrivals_us, (size_t)a->n_arrivals * sizeof(i64), cudaMemcpyHostToDevice,
                       ctx->stream),
       "H2D arrivals");
    *d_arr = ctx->dArr.p;
    return SMILESS_OK;
}

}  // namespace

// ======================================================================================
// C ABI
// ======================================================================================
extern "C" {

int smiless_create(smiless_ctx **out, int cuda_device, void *cuda_stream) {
    if (!out) {
        g_create_err = "out is NULL";
        return SMILESS_EINVAL;
    }
    *out = nullptr;
    if (cuda_device < 0) {
        g_create_err = "cuda_device must be >= 0";
        return SMILESS_EINVAL;
    }
    smiless_ctx *c = new (std::nothrow) smiless_ctx();
    if (!c) {
        g_create_err = "out of host memory";
        return SMILESS_ENOMEM;
    }
    c->device = cuda_device;
    c->stream = (cudaStream_t)cuda_stream;
    *out = c;
    return SMILESS_OK;
}

int smiless_set_stream(smiless_ctx *ctx, void *cuda_stream) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->stream = (cudaStream_t)cuda_stream;
    return SMILESS_OK;
}

void smiless_destroy(smiless_ctx *ctx) {
    if (!ctx) return;
    if (ctx->dev_ready) {
        cudaSetDevice(ctx->device);
        for (auto &kv : ctx->jit_cache)
            if (kv.second.mod) driver().moduleUnload(kv.second.mod);
        ctx->dI.release(); ctx->dNI.release(); ctx->dT.release(); ctx->dU.release(); ctx->dPtr.release(); ctx->dIdx.release();
        ctx->dArr.release(); ctx->dOff.release(); ctx->dScal.release(); ctx->dRrem.release(); ctx->dErr.release();
        ctx->dCounter.release(); ctx->dStats.release(); ctx->dInc.release(); ctx->dBlk.release(); ctx->dIdxEval.release();
        ctx->dCost.release(); ctx->dLat.release(); ctx->dFeas.release(); ctx->dRes.release(); ctx->dDump.release();
        ctx->dList.release(); ctx->dListCnt.release(); ctx->dW.release();
        ctx->dListA.release(); ctx->dListCntA.release(); ctx->dChunkCnt.release(); ctx->dListKeyA.release();
        ctx->dListM.release(); ctx->dListCntM.release(); ctx->dChunkCntM.release(); ctx->dDig.release();
        ctx->dCostList.release(); ctx->dCostN.release();
        ctx->dX.release(); ctx->dRecNx.release(); ctx->dRecNlu.release(); ctx->dRecPre.release();
        if (ctx->hRes) cudaFreeHost(ctx->hRes);
        for (auto &ev : ctx->ev)
            if (ev) cudaEventDestroy(ev);
    }
    delete ctx;
}

const char *smiless_last_error(const smiless_ctx *ctx) {
    if (!ctx) return g_create_err.c_str();
    return ctx->err.c_str();
}

int smiless_load_dag(smiless_ctx *ctx, int32_t n_funcs, const int32_t *pred_ptr, const int32_t *pred_idx) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (n_funcs < 1 || n_funcs > SMILESS_MAX_FUNCS)
        return fail(ctx, SMILESS_EINVAL, "n_funcs must be in [1, %d]", SMILESS_MAX_FUNCS);
    if (!pred_ptr) return fail(ctx, SMILESS_EINVAL, "pred_ptr is NULL");
    if (pred_ptr[0] != 0) return fail(ctx, SMILESS_EINVAL, "pred_ptr[0] must be 0");
    for (int k = 0; k < n_funcs; ++k)
        if (pred_ptr[k + 1] < pred_ptr[k]) return fail(ctx, SMILESS_EINVAL, "pred_ptr must be non-decreasing");
    const int E = pred_ptr[n_funcs];
    if (E > SMILESS_DEV_MAX_EDGES) return fail(ctx, SMILESS_EINVAL, "too many edges");
    if (E > 0 && !pred_idx) return fail(ctx, SMILESS_EINVAL, "pred_idx is NULL");
    u64 sinkmask = (n_funcs == 64) ? ~0ull : ((1ull << n_funcs) - 1);
    for (int k = 0; k < n_funcs; ++k) {
        u64 seen = 0;
        for (int e = pred_ptr[k]; e < pred_ptr[k + 1]; ++e) {
            const int p = pred_idx[e];
            if (p < 0 || p >= n_funcs) return fail(ctx, SMILESS_EINVAL, "pred_idx[%d] out of range", e);
            if (p >= k)
                return fail(ctx, SMILESS_ENOTTOPO, "function %d lists predecessor %d >= itself (not topological)", k, p);
            if ((seen >> p) & 1ull) return fail(ctx, SMILESS_EINVAL, "duplicate predecessor %d of %d", p, k);
            seen |= 1ull << p;
            sinkmask &= ~(1ull << p);
        }
    }
    ctx->N = n_funcs;
    ctx->pred_ptr.assign(pred_ptr, pred_ptr + n_funcs + 1);
    ctx->pred_idx.assign(pred_idx ? pred_idx : pred_ptr, pred_idx ? pred_idx + E : pred_ptr);
    ctx->sinkmask = sinkmask;
    ctx->dag_loaded = true;
    ctx->prof_loaded = false;  // profiles are per function: reload after a new DAG
    ctx->tables_dirty = true;
    return SMILESS_OK;
}

int smiless_load_profiles(smiless_ctx *ctx, const int32_t *n_configs, const int32_t *exec_us, const int32_t *init_us,
                          const double *price_per_us) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!ctx->dag_loaded) return fail(ctx, SMILESS_ESTATE, "load_dag first");
    if (!n_configs || !exec_us || !init_us || !price_per_us) return fail(ctx, SMILESS_EINVAL, "NULL profile array");
    int sum = 0;
    std::vector<int32_t> M(ctx->N), row0(ctx->N);
    for (int k = 0; k < ctx->N; ++k) {
        if (n_configs[k] < 1 || n_configs[k] > SMILESS_MAX_CONFIGS)
            return fail(ctx, SMILESS_EINVAL, "n_configs[%d] must be in [1, %d]", k, SMILESS_MAX_CONFIGS);
        M[k] = n_configs[k];
        row0[k] = sum;
        sum += n_configs[k];
    }
    i64 tmax = 0, imax = 0;
    for (int r = 0; r < sum; ++r) {
        if (exec_us[r] < 0 || exec_us[r] >= (1 << 29)) return fail(ctx, SMILESS_EINVAL, "exec_us[%d] out of [0, 2^29)", r);
        if (init_us[r] < 0 || init_us[r] >= (1 << 29)) return fail(ctx, SMILESS_EINVAL, "init_us[%d] out of [0, 2^29)", r);
        // -0.0 is rejected too: the kernels take the first cost term as is, so its sign bit
        // would make the cost bits order wrongly against the oracle's 0.0 + term
        if (!std::isfinite(price_per_us[r]) || price_per_us[r] < 0 || std::signbit(price_per_us[r]))
            return fail(ctx, SMILESS_EINVAL, "price_per_us[%d] must be finite and >= +0.0", r);
        tmax = std::max<i64>(tmax, init_us[r]);
        imax = std::max<i64>(imax, exec_us[r]);
    }
    ctx->M = M;
    ctx->row0 = row0;
    ctx->sumM = sum;
    ctx->I.assign(exec_us, exec_us + sum);
    ctx->T.assign(init_us, init_us + sum);
    ctx->U.assign(price_per_us, price_per_us + sum);
    ctx->Tmax = tmax;
    ctx->Imax = imax;
    ctx->prof_loaded = true;
    ctx->tables_dirty = true;
    return SMILESS_OK;
}

int smiless_space_size(const smiless_ctx *ctx, int32_t n_windows, int32_t n_fixed, uint64_t *out) {
    if (!ctx || !out) return SMILESS_EINVAL;
    if (!ctx->dag_loaded || !ctx->prof_loaded) return SMILESS_ESTATE;
    if (n_windows < 1 || n_windows > SMILESS_MAX_WINDOWS || n_fixed < 0 || n_fixed > ctx->N) return SMILESS_EINVAL;
    u64 s;
    if (!space_size_of(ctx, n_windows, n_fixed, &s)) return SMILESS_ERANGE;
    *out = s;
    return SMILESS_OK;
}

int smiless_decode(const smiless_ctx *ctx, int32_t n_windows, uint64_t index, const smiless_plan_args *a,
                   int32_t *config_out, int32_t *window_out) {
    if (!ctx || !config_out || !window_out) return SMILESS_EINVAL;
    if (!ctx->dag_loaded || !ctx->prof_loaded) return SMILESS_ESTATE;
    const int nf = a ? a->n_fixed : 0;
    if (n_windows < 1 || n_windows > SMILESS_MAX_WINDOWS || nf < 0 || nf > ctx->N) return SMILESS_EINVAL;
    if (nf > 0 && !a->fixed_digits) return SMILESS_EINVAL;
    u64 space;
    if (!space_size_of(ctx, n_windows, nf, &space)) return SMILESS_ERANGE;
    if (index >= space) return SMILESS_ERANGE;
    for (int k = ctx->N - 1; k >= nf; --k) {
        const u64 radix = (u64)ctx->M[k] * (u64)n_windows;
        const u64 d = index % radix;
        index /= radix;
        config_out[k] = (int32_t)(d / (u64)n_windows);
        window_out[k] = (int32_t)(d % (u64)n_windows);
    }
    for (int k = 0; k < nf; ++k) {
        if (a->fixed_digits[k] < 0 || (i64)a->fixed_digits[k] >= (i64)ctx->M[k] * n_windows) return SMILESS_EINVAL;
        config_out[k] = a->fixed_digits[k] / n_windows;
        window_out[k] = a->fixed_digits[k] % n_windows;
    }
    return SMILESS_OK;
}

int smiless_evaluate(smiless_ctx *ctx, const smiless_plan_args *a, const uint64_t *idx, int64_t n, double *cost,
                     int64_t *max_latency_us, uint8_t *feasible) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    int rc = validate_args(ctx, a, true);
    if (rc) return rc;
    if (n < 0 || (n > 0 && (!idx || !cost || !max_latency_us || !feasible)))
        return fail(ctx, SMILESS_EINVAL, "bad output arrays");
    u64 space;
    space_size_of(ctx, a->n_windows, a->n_fixed, &space);
    for (i64 i = 0; i < n; ++i)
        if (idx[i] >= space) return fail(ctx, SMILESS_ERANGE, "index %llu outside the space", (unsigned long long)idx[i]);
    if (n == 0) return SMILESS_OK;
    if ((rc = ensure_device(ctx))) return rc;
    CK(cudaSetDevice(ctx->device), "cudaSetDevice");
    if ((rc = upload_tables(ctx))) return rc;
    const i64 *d_arr = nullptr;
    if ((rc = stage_arrivals(ctx, a, &d_arr))) return rc;
    if ((rc = stage_row_windows(ctx, a))) return rc;
    CK(ctx->dIdxEval.ensure((size_t)n), "cudaMalloc");
    CK(ctx->dCost.ensure((size_t)n), "cudaMalloc");
    CK(ctx->dLat.ensure((size_t)n), "cudaMalloc");
    CK(ctx->dFeas.ensure((size_t)n), "cudaMalloc");
    CK(cudaMemcpyAsync(ctx->dIdxEval.p, idx, (size_t)n * 8, cudaMemcpyHostToDevice, ctx->stream), "H2D idx");
    ExactParams ep;
    fill_exact_params(ctx, a, d_arr, ep);
    ep.idx = ctx->dIdxEval.p;
    ep.n = n;
    ep.cost = ctx->dCost.p;
    ep.maxlat = (long long *)ctx->dLat.p;
    ep.feas = ctx->dFeas.p;
    ep.idx_from_res = 0;
    int e = smiless_dev_eval_exact(&ep, ctx->stream);
    if (e) return cuda_fail(ctx, (cudaError_t)e, "eval_exact launch");
    CK(cudaMemcpyAsync(cost, ctx->dCost.p, (size_t)n * 8, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
    CK(cudaMemcpyAsync(max_latency_us, ctx->dLat.p, (size_t)n * 8, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
    CK(cudaMemcpyAsync(feasible, ctx->dFeas.p, (size_t)n, cudaMemcpyDeviceToHost, ctx->stream), "D2H");
    CK(cudaStreamSynchronize(ctx->stream), "evaluate");
    return SMILESS_OK;
}

}  // extern "C"

namespace {

// NVTX range for the profilers (nsys / ncu --nvtx): the stages of a plan call (header-only
// nvtx3; a no-op unless a tool injects itself)
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

// SMILESS_PROFILE_HOST=1: host-side stage timestamps of every plan call on stderr (tuning aid)
struct HostProf {
    bool on;
    std::chrono::steady_clock::time_point t0, last;
    std::string line;
    HostProf() : on(getenv("SMILESS_PROFILE_HOST") != nullptr) {
        if (on) t0 = last = std::chrono::steady_clock::now();
    }
    void note(const char *what, unsigned long long v) {
        if (!on) return;
        char b[96];
        snprintf(b, sizeof b, " %s=%llu", what, v);
        line += b;
    }
    void mark(const char *what) {
        if (!on) return;
        const auto now = std::chrono::steady_clock::now();
        char b[96];
        snprintf(b, sizeof b, " %s=%.0fus", what, std::chrono::duration<double, std::micro>(now - last).count());
        line += b;
        last = now;
    }
    ~HostProf() {
        if (on)
            fprintf(stderr, "[smiless host] total=%.0fus%s\n",
                    std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count(),
                    line.c_str());
    }
};

// The hot path.  n_sla = 1: an ordinary plan with a->sla_us.  n_sla > 1: one evaluation of the
// space, one argmin key per SLA in slas[] (pruning against their maximum); a->sla_us is ignored.
// d_end > d_begin (smiless_plan_digits): plan the sub-spaces of every value d in [d_begin, d_end) of
// the last pinned digit one after the other inside this call -- arrivals, tables and the kernel
// staged once, the incumbent kept on the device from one digit to the next, each digit's winner
// reduced into its own slot, one exact re-check of the overall (cost, digit, index) minimum.
int plan_impl(smiless_ctx *ctx, const smiless_plan_args *a_in, const i64 *slas, int n_sla, smiless_plan_result *res,
              int32_t *config_out, int32_t *window_out, int32_t d_begin = 0, int32_t d_end = 0,
              int32_t *digit_out = nullptr) {
    if (!a_in) return fail(ctx, SMILESS_EINVAL, "args is NULL");
    HostProf hp;
    NvtxRange nv_plan("smiless_plan");
    ctx->h2d = ctx->d2h = 0;
    smiless_plan_args a_copy = *a_in;
    i64 sla_max = slas[0];
    for (int s_ = 1; s_ < n_sla; ++s_) sla_max = std::max<i64>(sla_max, slas[s_]);
    a_copy.sla_us = sla_max;
    const smiless_plan_args *a = &a_copy;
    const bool digit_mode = d_end > d_begin;
    int32_t fixed_local[SMILESS_MAX_FUNCS] = {0};
    if (digit_mode) {
        if (n_sla != 1) return fail(ctx, SMILESS_EINVAL, "digit ranges take one SLA");
        if (a->n_fixed < 1 || a->n_fixed >= ctx->N || !a->fixed_digits)
            return fail(ctx, SMILESS_EINVAL, "digit ranges need 1 <= n_fixed < n_funcs and fixed_digits");
        if (a->cost_out) return fail(ctx, SMILESS_EINVAL, "cost_out is not supported with digit ranges");
        const int32_t radix = ctx->M[a->n_fixed - 1] * a->n_windows;
        if (d_begin < 0 || d_end > radix)
            return fail(ctx, SMILESS_EINVAL, "digit range [%d, %d) outside [0, %d)", d_begin, d_end, radix);
        for (int k = 0; k < a->n_fixed; ++k) fixed_local[k] = a->fixed_digits[k];
        fixed_local[a->n_fixed - 1] = d_begin;
        a_copy.fixed_digits = fixed_local;
    }
    int rc = validate_args(ctx, a, true);
    if (rc) return rc;
    for (int s_ = 0; s_ < n_sla; ++s_)
        if (slas[s_] < 0 || slas[s_] >= (1ll << 29)) return fail(ctx, SMILESS_EINVAL, "sla out of [0, 2^29)");
    if (n_sla > 1 && (a->flags & SMILESS_FLAG_COST_CAP))
        return fail(ctx, SMILESS_EINVAL, "FLAG_COST_CAP is not supported by the SLA sweep");
    ctx->nsla = n_sla;
    struct NslaReset { smiless_ctx *c; ~NslaReset() { c->nsla = 1; } } nsla_reset{ctx};
    u64 space;
    space_size_of(ctx, a->n_windows, a->n_fixed, &space);
    const u64 cb = a->begin;
    const u64 ce = (a->end == 0 || a->end > space) ? space : a->end;
    if (cb > ce) return fail(ctx, SMILESS_EINVAL, "begin > end");
    if (a->cost_out && ce - cb > ((u64)1 << 26)) return fail(ctx, SMILESS_EINVAL, "cost_out range larger than 2^26");
    const int n_shards = a->n_shards <= 0 ? 1 : a->n_shards;
    const int shard = a->n_shards <= 0 ? 0 : a->shard;
    if ((rc = ensure_device(ctx))) return rc;
    CK(cudaSetDevice(ctx->device), "cudaSetDevice");
    if ((rc = upload_tables(ctx))) return rc;
    cudaStream_t st = ctx->stream;
    CK(cudaEventRecord(ctx->ev[0], st), "event");
    int launches = 0;
    int32_t eval_path = SMILESS_PATH_NONE;

    const i64 *d_arr = nullptr;
    if ((rc = stage_arrivals(ctx, a, &d_arr))) return rc;
    if ((rc = stage_row_windows(ctx, a))) return rc;

    const RangePlan rp = range_plan(ctx, a);
    const i64 n_steps = a->n_arrivals - 1;
    const i64 n_off = std::max<i64>(4, (n_steps + rp.K - 1) / rp.K * rp.K);
    const size_t tsz = rp.time64 ? 8 : 4;
    CK(ctx->dOff.ensure((size_t)n_off * tsz), "cudaMalloc offsets");
    CK(cudaMemsetAsync(ctx->dErr.p, 0, sizeof(int), st), "memset");
    CK(cudaMemsetAsync(ctx->dRes.p, 0xff, sizeof(ResBlock) * n_sla, st), "memset");
    CK(ctx->dRrem.ensure((size_t)(n_off / rp.K + 1)), "cudaMalloc rrem");
    int e = smiless_dev_prep_offsets(d_arr, a->n_arrivals, rp.d_cap, rp.K, rp.time64 ? 1 : 0, ctx->dOff.p, n_off,
                                     ctx->dScal.p, ctx->dErr.p, ctx->dRrem.p, st);
    if (e) return cuda_fail(ctx, (cudaError_t)e, "prep_offsets launch");
    ++launches;
    if (inst_mode(ctx, a)) {
        e = smiless_dev_prep_tail(d_arr, a->n_arrivals, rp.d_cap, rp.K, ctx->dScal.p, st);
        if (e) return cuda_fail(ctx, (cudaError_t)e, "prep_tail launch");
    }

    const bool single = a->n_fixed == ctx->N;    // nothing left to search: one candidate
    u64 digit_dec_lo = 0, digit_dec_hi = 0, digit_full = 0;
    int32_t digit_best = -1;
    double eval_ms = 0.0;
    u64 n_decided = 0, n_full = 0;
    if (!single && ce > cb) {
        // pick the path first, then compile only the kernel families it needs
        const bool prune_mode = !(a->flags & SMILESS_FLAG_NO_PRUNE);
        const char *memo_env0 = getenv("SMILESS_MEMO");
        const bool memo_path = !prune_mode && a->n_fixed < ctx->N && (!memo_env0 || atoi(memo_env0) != 0) &&
                               !virt_sink(ctx, a) &&
                               smem_memo_up(ctx, rp, n_off) <= 227 * 1024 &&
                               smem_memo_var(ctx, a, rp, n_off) <= 227 * 1024;
        const bool bnb_path = !memo_path && bb_depth(ctx, a) > 0 && smem_bound_bytes(ctx, a, rp, n_off) <= 227 * 1024;
        const int families = memo_path ? (FAM_MEMO | FAM_PLAN) : (bnb_path ? (FAM_PLAN | FAM_BOUND) : FAM_PLAN);
        hp.mark("setup");
        JitKernel *jk = nullptr;
        {
            NvtxRange nv("nvrtc specialisation (cached)");
            if ((rc = get_kernel(ctx, a, rp, n_off, families, &jk))) return rc;
        }
        hp.mark("get_kernel");
        // one evaluation of [cb, ce) for the current pinned digits, its winner reduced into dst;
        // `first`: the first (or only) digit uploads the caller's cap as the incumbent and starts
        // the evaluator's event
        auto run_once = [&](ResBlock *dst, const bool first) -> int {
            const u64 V = unit_cands(ctx, a);   // candidates per unit
            const u64 ub = cb / V, ue = (ce + V - 1) / V;
            const u64 U = ue - ub;
            const u64 n_chunks = (U + kChunkUnits - 1) / kChunkUnits;
            const u64 my_chunks = n_chunks > (u64)shard ? (n_chunks - 1 - (u64)shard) / (u64)n_shards + 1 : 0;
            const u64 claims_total = my_chunks * (u64)kChunkUnits;
            const int grid = jk->blocks_per_sm * ctx->n_sms;
            int grid_used = grid;                        // CTAs whose argmin slots the reduce reads
            CK(ctx->dBlk.ensure((size_t)grid * 2 * n_sla), "cudaMalloc");
            CK(cudaMemsetAsync(ctx->dBlk.p, 0xff, (size_t)grid * 16 * n_sla, st), "memset");
            CK(cudaMemsetAsync(ctx->dStats.p, 0, 16, st), "memset");
            PlanParamsHost pp;
            memset(&pp, 0, sizeof pp);
            pp.tabI = ctx->dI.p;
            pp.tabNI = ctx->dNI.p;
            pp.tabW = ctx->dW.p;
            pp.zero = 0;
            pp.tabT = ctx->dT.p;
            pp.tabU = ctx->dU.p;
            pp.off = ctx->dOff.p;
            pp.scal = ctx->dScal.p;
            pp.counter = ctx->dCounter.p;
            pp.stats = ctx->dStats.p;
            pp.blk_best = ctx->dBlk.p;
            pp.unit_begin = ub;
            pp.unit_end = ue;
            pp.cand_begin = cb;
            pp.cand_end = ce;
            pp.n_steps = n_steps;
            pp.n_off = n_off;
            pp.sumM = kernel_rows(ctx, a);
            pp.sla = (int)a->sla_us;
            for (int s_ = 0; s_ < n_sla; ++s_) pp.slas[s_] = (int)slas[s_];
            pp.prune = (a->flags & SMILESS_FLAG_NO_PRUNE) ? 0 : 1;
            // cost-bound pruning against a running incumbent (one SLA, no per-candidate dump);
            // SMILESS_COST_PRUNE=0 disables it
            {
                const char *cp_env = getenv("SMILESS_COST_PRUNE");
                pp.cost_prune = (pp.prune && n_sla == 1 && !a->cost_out && (!cp_env || atoi(cp_env) != 0)) ? 1 : 0;
                pp.inc = ctx->dInc.p;
                pp.rrem = ctx->dRrem.p;
                pp.cap = ~0ull;
                if (a->flags & SMILESS_FLAG_COST_CAP) {
                    double c = a->cost_cap + 0.0;               // -0.0 -> +0.0: bits order like the costs
                    memcpy(&pp.cap, &c, 8);
                }
                if (first) {                                   // later digits keep the running incumbent
                    CK(cudaMemcpyAsync(ctx->dInc.p, &pp.cap, 8, cudaMemcpyHostToDevice, st), "H2D incumbent");
                    ctx->h2d += 8;
                }
            }
            pp.shard = shard;
            pp.n_shards = n_shards;
            pp.chunk_units = kChunkUnits;
            for (int k = 0; k < a->n_fixed; ++k) pp.fixed[k] = a->fixed_digits[k];
            if (a->cost_out) {
                CK(ctx->dDump.ensure((size_t)(ce - cb)), "cudaMalloc dump");
                CK(cudaMemsetAsync(ctx->dDump.p, 0xff, (size_t)(ce - cb) * sizeof(double), st), "memset dump");  // NaN
                pp.dump = ctx->dDump.p;
            }
            const int D = bb_depth(ctx, a);
            pp.list_upp = 1;
            const bool memo = memo_path && jk->blocks_up > 0 && jk->blocks_var > 0;
            if (memo && jk->fn_fused) {
                eval_path = SMILESS_PATH_MEMO_FUSED;
                // ---- fused memoisation: upstream walked by each CTA's producer warp into a shared-
                // memory ring, variants by its consumer warps (evaluator.cuh smiless_fused_kernel);
                // split cost: the units holding a feasible candidate are re-walked by the plan
                // kernel in list mode (upstream recomputed per lane, sums of u, cost, argmin)
                const u64 upp = (u64)(ctx->M[ctx->N - 1] / configs_per_lane(ctx, a));
                const u64 pl0 = ub / upp, ph0 = (ue + upp - 1) / upp;
                const bool split = split_cost();
                // prefix batches bound the cost list; tiles of a batch are interleaved over the shards
                const u64 batch_p = std::min<u64>((u64)1 << 20, ph0 - pl0);
                if (split) {
                    CK(ctx->dCostList.ensure((size_t)(batch_p * upp)), "cudaMalloc cost list");
                    CK(ctx->dCostN.ensure(1), "cudaMalloc");
                }
                MemoParamsHost mp;
                memset(&mp, 0, sizeof mp);
                mp.tabNI = ctx->dNI.p;
                mp.tabT = ctx->dT.p;
                mp.tabW = ctx->dW.p;
                mp.tabU = ctx->dU.p;
                mp.off = ctx->dOff.p;
                mp.scal = ctx->dScal.p;
                mp.counter = ctx->dCounter.p;
                mp.stats = ctx->dStats.p;
                mp.cost_list = ctx->dCostList.p;
                mp.cost_n = ctx->dCostN.p;
                mp.dump = pp.dump;
                mp.cand_begin = cb;
                mp.cand_end = ce;
                mp.n_steps = n_steps;
                mp.n_off = n_off;
                mp.sumM = ctx->sumM;
                mp.sla = (int)a->sla_us;
                mp.zero = 0;
                mp.shard = shard;
                mp.n_shards = n_shards;
                for (int s_ = 0; s_ < n_sla; ++s_) mp.slas[s_] = (int)slas[s_];
                for (int k = 0; k < a->n_fixed; ++k) mp.fixed[k] = a->fixed_digits[k];
                const int grid_f = jk->blocks_fused * ctx->n_sms;
                if (grid_f > grid) {     // per-CTA argmin slots of the fused kernel
                    CK(ctx->dBlk.ensure((size_t)grid_f * 2 * n_sla), "cudaMalloc");
                    CK(cudaMemsetAsync(ctx->dBlk.p, 0xff, (size_t)grid_f * 16 * n_sla, st), "memset");
                    pp.blk_best = ctx->dBlk.p;
                }
                mp.blk_best = ctx->dBlk.p;
                // the cost re-walk: plan kernel, list mode over the fused pass's cost list
                PlanParamsHost pc = pp;
                pc.prune = 0;
                pc.cost_prune = 0;
                pc.cap = ~0ull;
                pc.horizon = 0;
                pc.claims_begin = 0;
                pc.claims_end = ~0ull;
                pc.list_in = ctx->dCostList.p;
                pc.list_n = ctx->dCostN.p;
                pc.list_upp = 1;
                pc.list_base = 0;
                pc.list_in_cap = batch_p * upp;
                pc.no_count = 1;
                if (first) CK(cudaEventRecord(ctx->ev[1], st), "event");
                NvtxRange nv("memo: fused producer/consumer batches");
                for (u64 b0 = pl0; b0 < ph0; b0 += batch_p) {
                    const u64 b1 = std::min(ph0, b0 + batch_p);
                    mp.pref_begin = b0;
                    mp.pref_end = b1;
                    mp.unit_begin = std::max(ub, b0 * upp);
                    mp.unit_end = std::min(ue, b1 * upp);
                    CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                    if (split) CK(cudaMemsetAsync(ctx->dCostN.p, 0, sizeof(unsigned), st), "memset cost list");
                    void *args[] = {&mp};
                    CUresult r = driver().launchKernel(jk->fn_fused, (unsigned)grid_f, 1, 1, fused_threads(), 1, 1,
                                                       (unsigned)jk->smem_fused, (CUstream)st, args, nullptr);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "fused launch");
                    ++launches;
                    if (split) {
                        CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                        void *cargs[] = {&pc};
                        r = driver().launchKernel(jk->fn, (unsigned)grid, 1, 1, kThreads, 1, 1, (unsigned)jk->smem,
                                                  (CUstream)st, cargs, nullptr);
                        if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "fused cost re-walk launch");
                        ++launches;
                    }
                }
                grid_used = std::max(grid, grid_f);
            } else if (memo) {
                eval_path = SMILESS_PATH_MEMO;
                // ---- prefix memoisation: upstream once per prefix, then the variants per unit ---------
                const u64 upp = (u64)(ctx->M[ctx->N - 1] / configs_per_lane(ctx, a));
                const u64 pl0 = ub / upp, ph0 = (ue + upp - 1) / upp;
                const size_t tsz2 = rp.time64 ? 8 : 4;
                // + SM_XPF + 1 groups of 4 steps of read-ahead slack for the variants kernel
                const size_t row_bytes = tsz2 * (size_t)(n_off + 4 * (xpf_groups() + 1));
                // Batches of up to 2^20 prefixes (fewer launches, fewer tails, a fuller upstream
                // kernel: 3.80e8 -> 3.95e8 candidates/s on the C2 slice, profiles/r02l_memo_batch.md),
                // the x buffer bounded by a quarter of the device memory; halved while the
                // allocation fails.  SMILESS_MEMO_BATCH (tuning) sets the prefixes per batch.
                size_t mem_free = 0, mem_total = 0;
                CK(cudaMemGetInfo(&mem_free, &mem_total), "cudaMemGetInfo");
                u64 max_batch = std::max<u64>(1, std::min<u64>((u64)1 << 20, (u64)(mem_total / 4) / row_bytes));
                if (const char *mb_env = getenv("SMILESS_MEMO_BATCH"))
                    max_batch = std::max<u64>(1, std::min<u64>((u64)atoll(mb_env), ((u64)64 << 30) / row_bytes));
                u64 batch_p = std::min<u64>(max_batch, ph0 - pl0);
                while (ctx->dX.ensure((size_t)batch_p * row_bytes) != cudaSuccess && batch_p > 1) {
                    cudaGetLastError();                                  // clear the allocation failure
                    batch_p = (batch_p + 1) / 2;
                }
                CK(ctx->dX.ensure((size_t)batch_p * row_bytes), "cudaMalloc memo buffer");
                CK(ctx->dRecNx.ensure((size_t)batch_p), "cudaMalloc");
                CK(ctx->dRecNlu.ensure((size_t)batch_p), "cudaMalloc");
                CK(ctx->dRecPre.ensure((size_t)batch_p), "cudaMalloc");
                if (jk->fn_varc) {
                    CK(ctx->dCostList.ensure((size_t)(batch_p * upp)), "cudaMalloc cost list");
                    CK(ctx->dCostN.ensure(1), "cudaMalloc");
                }
                MemoParamsHost mp;
                memset(&mp, 0, sizeof mp);
                mp.tabNI = ctx->dNI.p;
                mp.tabT = ctx->dT.p;
                mp.tabW = ctx->dW.p;
                mp.tabU = ctx->dU.p;
                mp.off = ctx->dOff.p;
                mp.scal = ctx->dScal.p;
                mp.counter = ctx->dCounter.p;
                mp.stats = ctx->dStats.p;
                mp.blk_best = ctx->dBlk.p;
                mp.xbuf = ctx->dX.p;
                mp.rec_nx = ctx->dRecNx.p;
                mp.rec_pre = ctx->dRecPre.p;
                mp.rec_nlu = ctx->dRecNlu.p;
                mp.cost_list = ctx->dCostList.p;
                mp.cost_n = ctx->dCostN.p;
                mp.dump = pp.dump;
                mp.cand_begin = cb;
                mp.cand_end = ce;
                mp.n_steps = n_steps;
                mp.n_off = n_off;
                mp.sumM = ctx->sumM;
                mp.sla = (int)a->sla_us;
                mp.zero = 0;
                for (int s_ = 0; s_ < n_sla; ++s_) mp.slas[s_] = (int)slas[s_];
                for (int k = 0; k < a->n_fixed; ++k) mp.fixed[k] = a->fixed_digits[k];
                const int grid_up = jk->blocks_up * ctx->n_sms;
                const int grid_var = jk->blocks_var * ctx->n_sms;
                if (grid_var > grid) {     // per-CTA argmin slots of the variants kernel
                    CK(ctx->dBlk.ensure((size_t)grid_var * 2 * n_sla), "cudaMalloc");
                    CK(cudaMemsetAsync(ctx->dBlk.p, 0xff, (size_t)grid_var * 16 * n_sla, st), "memset");
                    mp.blk_best = ctx->dBlk.p;
                }
                if (first) CK(cudaEventRecord(ctx->ev[1], st), "event");
                NvtxRange nv("memo: upstream + variants batches");
                u64 bi = 0;
                for (u64 b0 = pl0; b0 < ph0; b0 += batch_p, ++bi) {
                    if (bi % (u64)n_shards != (u64)shard) continue;
                    const u64 b1 = std::min(ph0, b0 + batch_p);
                    mp.pref_begin = b0;
                    mp.pref_end = b1;
                    mp.unit_begin = std::max(ub, b0 * upp);
                    mp.unit_end = std::min(ue, b1 * upp);
                    CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                    void *args[] = {&mp};
                    CUresult r = driver().launchKernel(jk->fn_up, (unsigned)grid_up, 1, 1, kThreads, 1, 1,
                                                       (unsigned)jk->smem_up, (CUstream)st, args, nullptr);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "upstream launch");
                    ++launches;
                    CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                    if (jk->fn_varc) CK(cudaMemsetAsync(ctx->dCostN.p, 0, sizeof(unsigned), st), "memset cost list");
                    r = driver().launchKernel(jk->fn_var, (unsigned)grid_var, 1, 1, vthreads_per_cta(), 1, 1,
                                              (unsigned)jk->smem_var, (CUstream)st, args, nullptr);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "variants launch");
                    ++launches;
                    if (jk->fn_varc) {                 // split cost: re-walk the units with a feasible candidate
                        CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                        r = driver().launchKernel(jk->fn_varc, (unsigned)grid_var, 1, 1, vthreads_per_cta(), 1, 1,
                                                  (unsigned)jk->smem_var, (CUstream)st, args, nullptr);
                        if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "variants cost launch");
                        ++launches;
                    }
                }
                grid_used = std::max(grid, grid_var);
            } else if (bnb_path && D > 0 && jk->blocks_bound > 0) {
                eval_path = SMILESS_PATH_BNB;
                // ---- exact branch-and-bound: prefixes of functions n_fixed..D-1, then list mode ----
                // Sharding (multi-GPU): the deep level's prefixes (one level) or the deep children of
                // every shallow survivor (two levels) are interleaved over the shards, ordinal
                // c = c' * n_shards + shard, so every rank decides an equal share of every survivor's
                // subtree; the shallow level (<= 2^22 prefixes) is replicated on every rank.
                const u64 S = cands_per_prefix(ctx, a, D);
                const u64 upp = S / V;                            // evaluator units per prefix
                const u64 p_lo = cb / S, p_hi = (ce + S - 1) / S;
                const u64 batch = (u64)1 << 22;                   // prefixes per range-mode bound launch
                const int DA = bb_depth_a(ctx, a, D);
                const u64 R = DA > 0 ? cands_per_prefix(ctx, a, DA) / S : 1;   // deep children per shallow prefix
                // deep survivor list: no launch enumerates more than list_cap ordinals, so it cannot
                // overflow (the kernel still checks, and a violation fails the call)
                u64 list_cap = R > ((u64)1 << 24) ? ((u64)1 << 26) : ((u64)1 << 24);
                if (const char *lc_env = getenv("SMILESS_BB_LISTCAP"))   // testing: force the split paths
                    list_cap = std::max<u64>(1, std::min<u64>(list_cap, (u64)atoll(lc_env)));
                CK(ctx->dList.ensure((size_t)list_cap), "cudaMalloc list");
                CK(ctx->dListCnt.ensure(1), "cudaMalloc");
                pp.list_in_cap = list_cap;
                BoundParamsHost bp;
                memset(&bp, 0, sizeof bp);
                bp.tabNI = ctx->dNI.p;
                bp.tabW = ctx->dW.p;
                bp.tabT = ctx->dT.p;
                bp.tabU = ctx->dU.p;
                bp.scal = ctx->dScal.p;
                bp.inc = ctx->dInc.p;
                bp.cost_prune = pp.cost_prune;
                bp.off = ctx->dOff.p;
                bp.counter = ctx->dCounter.p;
                bp.stats = ctx->dStats.p;
                bp.list_out = ctx->dList.p;
                bp.list_cnt = ctx->dListCnt.p;
                bp.list_cap = list_cap;
                bp.overflow = (unsigned *)ctx->dErr.p;            // bit 2 (value 4): list overflow
                bp.cands_per_prefix = S;
                bp.cand_begin = cb;
                bp.cand_end = ce;
                bp.n_steps = n_steps;
                bp.n_off = n_off;
                bp.sumM = kernel_rows(ctx, a);
                bp.sla = (int)a->sla_us;
                bp.zero = 0;
                bp.shard = shard;
                bp.n_shards = n_shards;
                bp.attr_shard = 0;
                bp.attr_n = 1;
                for (int k = 0; k < ctx->N; ++k) {
                    int m = ctx->I[ctx->row0[k]];
                    for (int c = 1; c < ctx->M[k]; ++c) m = std::min(m, ctx->I[ctx->row0[k] + c]);
                    bp.nimin[k] = -m;
                }
                for (int k = 0; k < a->n_fixed; ++k) bp.fixed[k] = a->fixed_digits[k];
                const int grid_b = jk->blocks_bound * ctx->n_sms;
                if (first) CK(cudaEventRecord(ctx->ev[1], st), "event");
                // evaluator over the deep survivors in dList (absolute depth-D prefix ids)
                auto run_eval = [&]() -> int {
                    CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                    pp.claims_begin = 0;
                    pp.claims_end = ~0ull;
                    pp.list_in = ctx->dList.p;
                    pp.list_n = ctx->dListCnt.p;
                    pp.list_upp = upp;
                    pp.list_base = 0;
                    pp.list_out = nullptr;
                    pp.list_cnt = nullptr;
                    pp.horizon = 0;
                    void *args[] = {&pp};
                    CUresult r = driver().launchKernel(jk->fn, (unsigned)grid, 1, 1, kThreads, 1, 1, (unsigned)jk->smem,
                                                       (CUstream)st, args, nullptr);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "evaluator launch");
                    ++launches;
                    return SMILESS_OK;
                };
                auto run_bound = [&](CUfunction fn) -> int {
                    void *bargs[] = {&bp};
                    CUresult r = driver().launchKernel(fn, (unsigned)grid_b, 1, 1, kThreads, 1, 1,
                                                       (unsigned)jk->smem_bound, (CUstream)st, bargs, nullptr);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "bound launch");
                    ++launches;
                    return SMILESS_OK;
                };
                if (DA > 0) {
                    // ---- two levels: depth DA over every prefix, depth D over the DA survivors' children --
                    const u64 SA = cands_per_prefix(ctx, a, DA);
                    const u64 a_lo = cb / SA, a_hi = (ce + SA - 1) / SA;
                    CK(ctx->dListA.ensure((size_t)batch), "cudaMalloc list");
                    CK(ctx->dListCntA.ensure(1), "cudaMalloc");
                    // best-first: with the cost bound on, the shallow survivors are sorted by their
                    // static cost lower bound so the first deep launch sets a good incumbent early
                    // (SMILESS_BB_SORT=1; off by default: measured slower on C2 with live windows and
                    // no faster elsewhere, profiles/r02k_bb_sort.md)
                    const char *sort_env = getenv("SMILESS_BB_SORT");
                    const bool bb_sort = pp.cost_prune && sort_env && atoi(sort_env) != 0;
                    if (bb_sort) CK(ctx->dListKeyA.ensure((size_t)batch), "cudaMalloc keys");
                    std::vector<u64> h_pref, h_key;
                    std::vector<uint32_t> h_ord;
                    for (u64 b0 = a_lo; b0 < a_hi; b0 += batch) {
                        const u64 b1 = std::min(a_hi, b0 + batch);
                        CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                        CK(cudaMemsetAsync(ctx->dListCntA.p, 0, sizeof(unsigned), st), "memset list");
                        bp.list_in = nullptr;
                        bp.list_n = nullptr;
                        bp.list_upp = 1;
                        bp.list_stride = 1;
                        bp.list_r0 = 0;
                        bp.prefix_begin = b0;
                        bp.prefix_end = b1;
                        bp.cands_per_prefix = SA;
                        bp.list_out = ctx->dListA.p;
                        bp.list_cnt = ctx->dListCntA.p;
                        bp.list_cap = batch;
                        bp.shard = 0;                                 // replicated on every shard ...
                        bp.n_shards = 1;
                        bp.attr_shard = shard;                        // ... its pruned prefixes counted once
                        bp.attr_n = n_shards;
                        bp.list_key = bb_sort ? ctx->dListKeyA.p : nullptr;
                        {
                            NvtxRange nv("bnb shallow level");
                            if ((rc = run_bound(jk->fn_bound_a))) return rc;
                        }
                        unsigned n_a = 0;
                        hp.mark("launch_a");
                        CK(cudaMemcpyAsync(&n_a, ctx->dListCntA.p, sizeof n_a, cudaMemcpyDeviceToHost, st), "D2H count");
                        ctx->d2h += sizeof n_a;
                        CK(cudaStreamSynchronize(st), "count");
                        hp.mark("sync_a");
                        hp.note("n_a", n_a);
                        bp.list_key = nullptr;
                        if (bb_sort && n_a > 1 && n_a <= (1u << 18)) {
                            // (key, prefix) ascending; ties by prefix: a deterministic order on every rank
                            h_pref.resize(n_a);
                            h_key.resize(n_a);
                            CK(cudaMemcpyAsync(h_pref.data(), ctx->dListA.p, n_a * sizeof(u64), cudaMemcpyDeviceToHost, st),
                               "D2H survivors");
                            CK(cudaMemcpyAsync(h_key.data(), ctx->dListKeyA.p, n_a * sizeof(u64), cudaMemcpyDeviceToHost, st),
                               "D2H keys");
                            CK(cudaStreamSynchronize(st), "survivors");
                            h_ord.resize(n_a);
                            for (uint32_t q = 0; q < n_a; ++q) h_ord[q] = q;
                            std::sort(h_ord.begin(), h_ord.end(), [&](uint32_t x, uint32_t y) {
                                return h_key[x] != h_key[y] ? h_key[x] < h_key[y] : h_pref[x] < h_pref[y];
                            });
                            std::vector<u64> sorted(n_a);
                            for (uint32_t q = 0; q < n_a; ++q) sorted[q] = h_pref[h_ord[q]];
                            CK(cudaMemcpyAsync(ctx->dListA.p, sorted.data(), n_a * sizeof(u64), cudaMemcpyHostToDevice, st),
                               "H2D survivors");
                            ctx->d2h += 2 * (u64)n_a * sizeof(u64);
                            ctx->h2d += (u64)n_a * sizeof(u64);
                            hp.mark("sort_a");
                        }
                        // Launches over a survivor list (first entry, entries, first child, children per
                        // entry): at most list_cap ordinals each.  With the cost bound on, the first launch
                        // is small and each next one SMILESS_BB_GROW (256) times larger: every launch's
                        // static prefix bound prunes against the incumbent the evaluations before it set,
                        // so the incumbent is refined before the bulk of the list (C2 at SLA 8 s:
                        // 131,072-entry chunks right after the 64-entry first one took 95-406 ms depending
                        // on which survivors came first, 113-137 ms with a 16,384-entry step between;
                        // profiles/r02p_bb_grow.md).  A survivor with more than list_cap children spans
                        // several.
                        struct DeepLaunch { u64 e0; unsigned ne; u64 r0, span; };
                        auto make_chunks = [&](u64 n_entries, u64 Rc) {
                            std::vector<DeepLaunch> L;
                            if (Rc <= list_cap) {
                                const u64 per_chunk = list_cap / Rc;
                                const char *first_env = getenv("SMILESS_BB_FIRST");
                                const u64 first = std::max<u64>(
                                    1, std::min<u64>(per_chunk,
                                                     pp.cost_prune ? (first_env ? (u64)atoll(first_env) : 64) : per_chunk));
                                const char *grow_env = getenv("SMILESS_BB_GROW");
                                const u64 grow = std::max<u64>(1, grow_env ? (u64)atoll(grow_env) : 256);
                                u64 cur = first;
                                for (u64 c0 = 0; c0 < n_entries;) {
                                    const u64 len = std::min<u64>(cur, n_entries - c0);
                                    L.push_back({c0, (unsigned)len, 0, Rc});
                                    c0 += len;
                                    cur = std::min<u64>(per_chunk, cur * grow);
                                }
                            } else {
                                for (u64 e = 0; e < n_entries; ++e)
                                    for (u64 r0 = 0; r0 < Rc; r0 += list_cap)
                                        L.push_back({e, 1u, r0, std::min(list_cap, Rc - r0)});
                            }
                            return L;
                        };
                        auto upload_counts = [&](const std::vector<DeepLaunch> &L, DevBuf<unsigned> &buf) -> int {
                            std::vector<unsigned> cnts(std::max<size_t>(L.size(), 1), 0u);
                            for (size_t i = 0; i < L.size(); ++i) cnts[i] = L[i].ne;
                            CK(buf.ensure(cnts.size()), "cudaMalloc counts");
                            ctx->h2d += cnts.size() * sizeof(unsigned);
                            CK(cudaMemcpyAsync(buf.p, cnts.data(), cnts.size() * sizeof(unsigned), cudaMemcpyHostToDevice, st),
                               "H2D counts");
                            return SMILESS_OK;
                        };
                        // one level over the children of a survivor list: bound kernel `fn` at depth with
                        // `Sc` candidates per prefix writes its survivors to out / out_cnt; then `after`
                        auto run_level = [&](CUfunction fn, const u64 *list, const std::vector<DeepLaunch> &L,
                                             DevBuf<unsigned> &cnt_buf, u64 Rc, u64 Sc, u64 *out, unsigned *out_cnt,
                                             int shard_, int n_shards_, const std::function<int(size_t)> &after) -> int {
                            for (size_t i = 0; i < L.size(); ++i) {
                                CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                                CK(cudaMemsetAsync(out_cnt, 0, sizeof(unsigned), st), "memset list");
                                bp.list_in = list + L[i].e0;
                                bp.list_n = cnt_buf.p + i;
                                bp.list_upp = L[i].span;
                                bp.list_stride = Rc;
                                bp.list_r0 = L[i].r0;
                                bp.prefix_begin = 0;
                                bp.prefix_end = 0;
                                bp.cands_per_prefix = Sc;
                                bp.list_out = out;
                                bp.list_cnt = out_cnt;
                                bp.list_cap = list_cap;
                                bp.shard = shard_;
                                bp.n_shards = n_shards_;
                                bp.attr_shard = 0;
                                bp.attr_n = 1;
                                if ((rc = run_bound(fn))) return rc;
                                if ((rc = after(i))) return rc;
                            }
                            return SMILESS_OK;
                        };
                        const int DM = jk->fn_bound_m ? bb_depth_m(ctx, a, D, DA) : 0;
                        if (DM == 0) {
                            // two levels: the deep children of the shallow survivors, interleaved over shards
                            const std::vector<DeepLaunch> L = make_chunks(n_a, R);
                            if ((rc = upload_counts(L, ctx->dChunkCnt))) return rc;
                            NvtxRange nv("bnb deep level + evaluate");
                            if ((rc = run_level(jk->fn_bound, ctx->dListA.p, L, ctx->dChunkCnt, R, S, ctx->dList.p,
                                                ctx->dListCnt.p, shard, n_shards, [&](size_t) { return run_eval(); })))
                                return rc;
                        } else {
                            // three levels: the middle children of the shallow survivors (interleaved over
                            // shards), then the deep children of each middle launch's survivors (this
                            // rank's own, not split again) and the evaluator over those
                            const u64 SMd = cands_per_prefix(ctx, a, DM);
                            const u64 R1 = SA / SMd, R2 = SMd / S;
                            CK(ctx->dListM.ensure((size_t)list_cap), "cudaMalloc list");
                            CK(ctx->dListCntM.ensure(1), "cudaMalloc");
                            const std::vector<DeepLaunch> Lm = make_chunks(n_a, R1);
                            if ((rc = upload_counts(Lm, ctx->dChunkCntM))) return rc;
                            NvtxRange nv("bnb middle + deep level + evaluate");
                            auto deep = [&](size_t) -> int {
                                unsigned n_m = 0;
                                CK(cudaMemcpyAsync(&n_m, ctx->dListCntM.p, sizeof n_m, cudaMemcpyDeviceToHost, st), "D2H count");
                                ctx->d2h += sizeof n_m;
                                CK(cudaStreamSynchronize(st), "count");
                                hp.note("n_m", n_m);
                                if (n_m == 0) return SMILESS_OK;
                                const std::vector<DeepLaunch> L = make_chunks(n_m, R2);
                                if ((rc = upload_counts(L, ctx->dChunkCnt))) return rc;
                                return run_level(jk->fn_bound, ctx->dListM.p, L, ctx->dChunkCnt, R2, S, ctx->dList.p,
                                                 ctx->dListCnt.p, 0, 1, [&](size_t) { return run_eval(); });
                            };
                            if ((rc = run_level(jk->fn_bound_m, ctx->dListA.p, Lm, ctx->dChunkCntM, R1, SMd, ctx->dListM.p,
                                                ctx->dListCntM.p, shard, n_shards, deep)))
                                return rc;
                        }
                        hp.mark("chunks_launched");
                        CK(cudaStreamSynchronize(st), "chunks");      // the next batch reuses dListA
                        hp.mark("sync_chunks");
                    }
                } else {
                    NvtxRange nv("bnb level + evaluate");
                    const u64 rbatch = std::min(batch, list_cap);     // a launch's survivors fit the list
                    for (u64 b0 = p_lo; b0 < p_hi; b0 += rbatch) {
                        const u64 b1 = std::min(p_hi, b0 + rbatch);
                        CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                        CK(cudaMemsetAsync(ctx->dListCnt.p, 0, sizeof(unsigned), st), "memset list");
                        bp.list_in = nullptr;
                        bp.list_n = nullptr;
                        bp.list_upp = 1;
                        bp.list_stride = 1;
                        bp.list_r0 = 0;
                        bp.prefix_begin = b0;
                        bp.prefix_end = b1;
                        if ((rc = run_bound(jk->fn_bound))) return rc;
                        if ((rc = run_eval())) return rc;
                    }
                }
            } else {
                eval_path = SMILESS_PATH_PLAN;
                // split very large ranges into several launches (bounded kernel duration).  Prune mode
                // with J - 1 > horizon runs each batch twice: pass 1 (every unit, `horizon` steps,
                // survivors compacted into a list), pass 2 (survivors only, all steps).
                const char *hz_env = getenv("SMILESS_HORIZON");
                i64 horizon = hz_env ? atoll(hz_env) : 128;
                horizon = horizon / rp.K * rp.K;
                const bool compact = pp.prune && horizon > 0 && horizon < n_steps;
                const u64 claims_per_launch = compact ? ((u64)1 << 24) : ((u64)1 << 28);   // units
                if (compact) {
                    CK(ctx->dList.ensure((size_t)claims_per_launch), "cudaMalloc list");
                    CK(ctx->dListCnt.ensure(1), "cudaMalloc");
                }
                if (first) CK(cudaEventRecord(ctx->ev[1], st), "event");
                NvtxRange nv("evaluate");
                for (u64 q0 = 0; q0 < claims_total; q0 += claims_per_launch) {
                    const u64 q1 = std::min(claims_total, q0 + claims_per_launch);
                    CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                    pp.claims_begin = q0;
                    pp.claims_end = q1;
                    pp.list_in = nullptr;
                    pp.list_n = nullptr;
                    pp.list_out = nullptr;
                    pp.list_cnt = nullptr;
                    pp.horizon = 0;
                    if (compact) {
                        CK(cudaMemsetAsync(ctx->dListCnt.p, 0, sizeof(unsigned), st), "memset list");
                        pp.list_out = ctx->dList.p;
                        pp.list_cnt = ctx->dListCnt.p;
                        pp.list_base = ub + (q0 / kChunkUnits * (u64)n_shards + (u64)shard) * kChunkUnits;
                        pp.list_in_cap = claims_per_launch;
                        pp.horizon = horizon;
                    }
                    void *args[] = {&pp};
                    CUresult r = driver().launchKernel(jk->fn, (unsigned)grid, 1, 1, kThreads, 1, 1, (unsigned)jk->smem,
                                                       (CUstream)st, args, nullptr);
                    if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "evaluator launch");
                    ++launches;
                    if (compact) {                                    // pass 2 over the survivors
                        CK(cudaMemsetAsync(ctx->dCounter.p, 0, 8, st), "memset counter");
                        pp.claims_begin = 0;
                        pp.claims_end = ~0ull;
                        pp.list_in = ctx->dList.p;
                        pp.list_n = ctx->dListCnt.p;
                        pp.list_out = nullptr;
                        pp.list_cnt = nullptr;
                        pp.horizon = 0;
                        r = driver().launchKernel(jk->fn, (unsigned)grid, 1, 1, kThreads, 1, 1, (unsigned)jk->smem,
                                                  (CUstream)st, args, nullptr);
                        if (r != CUDA_SUCCESS) return drv_fail(ctx, r, "evaluator launch");
                        ++launches;
                    }
                }
            }
            NvtxRange nv("argmin reduce");
            for (int s_ = 0; s_ < n_sla; ++s_) {
                int e2 = smiless_dev_reduce_best(ctx->dBlk.p + 2 * s_, grid_used, n_sla, dst + s_, st);
                if (e2) return cuda_fail(ctx, (cudaError_t)e2, "reduce launch");
                ++launches;
            }
            CK(cudaMemcpyAsync(&dst->stats[0], ctx->dStats.p, 16, cudaMemcpyDeviceToDevice, st), "D2D stats");
            if (a->cost_out) {
                ctx->d2h += (size_t)(ce - cb) * sizeof(double);
                CK(cudaMemcpyAsync(a->cost_out, ctx->dDump.p, (size_t)(ce - cb) * sizeof(double), cudaMemcpyDeviceToHost, st),
                   "D2H dump");
            }
            return SMILESS_OK;
        };
        if (!digit_mode) {
            if ((rc = run_once(ctx->dRes.p, true))) return rc;
        } else {
            const int n_dig = d_end - d_begin;
            CK(ctx->dDig.ensure((size_t)n_dig), "cudaMalloc digit results");
            for (int d = d_begin; d < d_end; ++d) {
                fixed_local[a->n_fixed - 1] = d;
                if ((rc = run_once(ctx->dDig.p + (d - d_begin), d == d_begin))) return rc;
            }
            // the lexicographic (cost bits, digit, index) minimum over the digits' winners; the
            // decided counts summed in 128 bits (C5: 128 digits x 2^63 candidates)
            std::vector<ResBlock> hd((size_t)n_dig);
            CK(cudaMemcpyAsync(hd.data(), ctx->dDig.p, sizeof(ResBlock) * (size_t)n_dig, cudaMemcpyDeviceToHost, st),
               "D2H digit results");
            ctx->d2h += sizeof(ResBlock) * (size_t)n_dig;
            CK(cudaStreamSynchronize(st), "digits");
            int best_d = -1;
            unsigned __int128 dec = 0;
            u64 full = 0;
            for (int i = 0; i < n_dig; ++i) {
                dec += hd[i].stats[0];
                full += hd[i].stats[1];
                if (hd[i].best_i == ~0ull) continue;
                if (best_d < 0 || hd[i].best_c < hd[best_d].best_c) best_d = i;   // ties: the lower digit
            }
            digit_dec_lo = (u64)dec;
            digit_dec_hi = (u64)(dec >> 64);
            digit_full = full;
            digit_best = best_d < 0 ? -1 : d_begin + best_d;
            fixed_local[a->n_fixed - 1] = best_d < 0 ? d_begin : d_begin + best_d;
            const u64 win[2] = {best_d < 0 ? ~0ull : hd[best_d].best_c, best_d < 0 ? ~0ull : hd[best_d].best_i};
            CK(cudaMemcpyAsync(&ctx->dRes.p->best_c, win, 16, cudaMemcpyHostToDevice, st), "H2D winner");
            ctx->h2d += 16;
        }
        CK(cudaEventRecord(ctx->ev[2], st), "event");
    } else if (single && ce > cb) {
        // the space is the single candidate of the pinned digits: index 0
        for (int s_ = 0; s_ < n_sla; ++s_) CK(cudaMemsetAsync(&ctx->dRes.p[s_].best_c, 0, 16, st), "memset");
        CK(cudaEventRecord(ctx->ev[1], st), "event");
        CK(cudaEventRecord(ctx->ev[2], st), "event");
    } else {
        CK(cudaEventRecord(ctx->ev[1], st), "event");
        CK(cudaEventRecord(ctx->ev[2], st), "event");
    }
    // a10: exact int64 re-evaluation of each winner (also decodes its digits), one thread per SLA
    {
        NvtxRange nv("exact winner re-check");
        ExactParams ep;
        fill_exact_params(ctx, a, d_arr, ep);
        for (int s_ = 0; s_ < n_sla; ++s_) ep.slas[s_] = slas[s_];
        ep.n = n_sla;
        ep.res = ctx->dRes.p;
        ep.idx_from_res = 1;
        e = smiless_dev_eval_exact(&ep, st);
        if (e) return cuda_fail(ctx, (cudaError_t)e, "eval_exact launch");
        ++launches;
    }
    CK(cudaMemcpyAsync(&ctx->dRes.p->err, ctx->dErr.p, sizeof(int), cudaMemcpyDeviceToDevice, st), "D2D err");
    CK(cudaMemcpyAsync(ctx->hRes, ctx->dRes.p, sizeof(ResBlock) * n_sla, cudaMemcpyDeviceToHost, st), "D2H result");
    ctx->d2h += sizeof(ResBlock) * n_sla;
    CK(cudaEventRecord(ctx->ev[3], st), "event");
    hp.mark("tail_launched");
    CK(cudaStreamSynchronize(st), "plan");
    hp.mark("sync_final");
    float ms = 0.f, tot = 0.f;
    cudaEventElapsedTime(&ms, ctx->ev[1], ctx->ev[2]);
    cudaEventElapsedTime(&tot, ctx->ev[0], ctx->ev[3]);
    eval_ms = ms;

    const ResBlock &h0 = *ctx->hRes;
    if (h0.err & 1) return fail(ctx, SMILESS_EINVAL, "arrivals must be non-decreasing");
    if (h0.err & 2) return fail(ctx, SMILESS_EINVAL, "arrival times out of range (|r| >= 2^62)");
    if (h0.err & 4) return fail(ctx, SMILESS_ECUDA, "internal: branch-and-bound survivor list overflow");
    if (!single && ce > cb) {
        n_decided = digit_mode ? digit_dec_lo : h0.stats[0];
        n_full = digit_mode ? digit_full : h0.stats[1];
    } else if (single && ce > cb) {
        n_decided = n_full = 1;
    }
    int status = SMILESS_INFEASIBLE;
    for (int s_ = 0; s_ < n_sla; ++s_) {
        const ResBlock &h = ctx->hRes[s_];
        const bool found = h.best_i != ~0ull && h.feasible == 1 &&
                           !((a->flags & SMILESS_FLAG_COST_CAP) && !(h.cost <= a->cost_cap + 0.0));
        if (!single && h.best_i != ~0ull && h.feasible != 1)
            return fail(ctx, SMILESS_ECUDA, "internal: evaluator winner %llu not feasible on exact re-evaluation",
                        (unsigned long long)h.best_i);
        if (found && !single) {
            double c;
            memcpy(&c, &h.best_c, 8);
            if (c != h.cost)
                return fail(ctx, SMILESS_ECUDA, "internal: evaluator cost %.17g != exact %.17g for index %llu", c,
                            h.cost, (unsigned long long)h.best_i);
        }
        smiless_plan_result &r = res[s_];
        memset(&r, 0, sizeof r);
        r.n_decided = n_decided;
        r.n_full_evals = n_full;
        r.eval_kernel_ms = eval_ms;
        r.total_device_ms = tot;
        r.int64_path = rp.time64 ? 1 : 0;
        r.launches = launches;
        r.h2d_bytes = ctx->h2d;
        r.d2h_bytes = ctx->d2h;
        r.eval_path = eval_path;
        r.n_decided_hi = digit_mode ? (uint32_t)digit_dec_hi : 0u;
        int32_t *co = config_out ? config_out + (size_t)s_ * ctx->N : nullptr;
        int32_t *wo = window_out ? window_out + (size_t)s_ * ctx->N : nullptr;
        if (!found) {
            r.index = ~0ull;
            r.cost = HUGE_VAL;
            r.max_latency_us = -1;
            for (int k = 0; k < ctx->N; ++k) {
                if (co) co[k] = -1;
                if (wo) wo[k] = -1;
            }
            continue;
        }
        if (s_ == 0) status = SMILESS_OK;
        if (digit_out) *digit_out = digit_mode ? digit_best : -1;
        r.index = h.best_i;
        r.cost = h.cost;
        r.max_latency_us = h.maxlat;
        for (int k = 0; k < ctx->N; ++k) {
            if (co) co[k] = h.cfg[k];
            if (wo) wo[k] = h.win[k];
        }
    }
    return status;
}

}  // namespace

extern "C" {

int smiless_plan(smiless_ctx *ctx, const smiless_plan_args *a, smiless_plan_result *res, int32_t *config_out,
                 int32_t *window_out) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!res) return fail(ctx, SMILESS_EINVAL, "res is NULL");
    if (!a) return fail(ctx, SMILESS_EINVAL, "args is NULL");
    const i64 sla = a->sla_us;
    return plan_impl(ctx, a, &sla, 1, res, config_out, window_out);
}

int smiless_plan_digits(smiless_ctx *ctx, const smiless_plan_args *a, int32_t d_begin, int32_t d_end,
                        smiless_plan_result *res, int32_t *digit_out, int32_t *config_out, int32_t *window_out) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!res) return fail(ctx, SMILESS_EINVAL, "res is NULL");
    if (!a) return fail(ctx, SMILESS_EINVAL, "args is NULL");
    if (d_end <= d_begin) return fail(ctx, SMILESS_EINVAL, "empty digit range [%d, %d)", d_begin, d_end);
    if (digit_out) *digit_out = -1;
    const i64 sla = a->sla_us;
    return plan_impl(ctx, a, &sla, 1, res, config_out, window_out, d_begin, d_end, digit_out);
}

int smiless_derive_windows(const smiless_ctx *ctx, int64_t it_us, int32_t *row_windows_out) {
    if (!ctx || !row_windows_out) return SMILESS_EINVAL;
    if (!ctx->dag_loaded || !ctx->prof_loaded) return SMILESS_ESTATE;
    if (it_us < 0) return SMILESS_EINVAL;
    for (int r = 0; r < ctx->sumM; ++r) {
        const i64 t = ctx->T[r], i = ctx->I[r];
        const i64 w = (t + i < it_us) ? it_us - t - i : 0;   // Case I gap, else Case II keep-alive
        row_windows_out[r] = (int32_t)std::min<i64>(w, (1 << 29) - 1);
    }
    return SMILESS_OK;
}

int smiless_top1_search(smiless_ctx *ctx, const smiless_plan_args *a, int64_t it_us, smiless_plan_result *res,
                        int32_t *config_out, int32_t *window_out, int64_t *n_nodes) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!a || !res) return fail(ctx, SMILESS_EINVAL, "args / res is NULL");
    if (!a->row_windows_us) return fail(ctx, SMILESS_EINVAL, "top1 search needs row_windows_us (n_windows == 1)");
    if (a->n_fixed != 0) return fail(ctx, SMILESS_EINVAL, "top1 search does not take pinned digits");
    int rc = validate_args(ctx, a, true);
    if (rc) return rc;
    const int N = ctx->N;
    // per-function ranking by the paper's per-invocation cost (Eq. 5 / Case II), ties: lower config
    std::vector<std::vector<int>> rank(N);
    std::vector<int> fastest(N);
    for (int k = 0; k < N; ++k) {
        std::vector<std::pair<double, int>> c;
        int fk = 0;
        for (int m = 0; m < ctx->M[k]; ++m) {
            const int row = ctx->row0[k] + m;
            const i64 t = ctx->T[row], i = ctx->I[row];
            const double per_inv = (t + i < it_us) ? (double)(t + i) : (double)it_us;
            c.push_back({ctx->U[row] * per_inv, m});
            if (ctx->I[row] < ctx->I[ctx->row0[k] + fk]) fk = m;
        }
        std::stable_sort(c.begin(), c.end(), [](const std::pair<double, int> &x, const std::pair<double, int> &y) {
            return x.first < y.first;
        });
        for (auto &pr : c) rank[k].push_back(pr.second);
        fastest[k] = fk;
    }
    auto index_of = [&](const std::vector<int> &cfg) {     // W == 1: digit = config
        u64 idx = 0;
        for (int k = 0; k < N; ++k) idx = idx * (u64)ctx->M[k] + (u64)cfg[k];
        return idx;
    };
    i64 nodes = 0;
    std::vector<int> chosen(N, -1);
    std::vector<u64> batch;
    std::vector<double> cost;
    std::vector<int64_t> lat;
    std::vector<uint8_t> feas;
    auto eval = [&](const std::vector<std::vector<int>> &cfgs) -> int {
        batch.clear();
        for (auto &c : cfgs) batch.push_back(index_of(c));
        cost.assign(batch.size(), 0.0);
        lat.assign(batch.size(), 0);
        feas.assign(batch.size(), 0);
        nodes += (i64)batch.size();
        return smiless_evaluate(ctx, a, (const uint64_t *)batch.data(), (int64_t)batch.size(), cost.data(), lat.data(),
                                feas.data());
    };
    // root T^0: every function on its cheapest configuration (Eq. 6)
    std::vector<int> root(N);
    for (int k = 0; k < N; ++k) root[k] = rank[k][0];
    if ((rc = eval({root}))) return rc;
    std::vector<int> leaf = root;
    bool ok = feas[0] != 0;
    if (!ok) {
        for (int k = 0; k < N; ++k) {
            std::vector<std::vector<int>> layer;
            const int r0 = (k == 0) ? 1 : 0;                // T^1_1: F_1 on its second cheapest
            for (int r = r0; r < ctx->M[k]; ++r) {
                std::vector<int> c(N);
                for (int q = 0; q < N; ++q) c[q] = q < k ? chosen[q] : (q == k ? rank[k][r] : fastest[q]);
                layer.push_back(c);
            }
            int pick = -1;
            if (!layer.empty()) {
                if ((rc = eval(layer))) return rc;
                for (size_t i = 0; i < layer.size(); ++i)
                    if (feas[i]) { pick = (int)i; break; }
            }
            chosen[k] = pick >= 0 ? layer[pick][k] : fastest[k];
        }
        leaf = chosen;
        if ((rc = eval({leaf}))) return rc;
        ok = feas[0] != 0;
    }
    memset(res, 0, sizeof *res);
    res->n_decided = (u64)nodes;
    res->n_full_evals = (u64)nodes;
    if (n_nodes) *n_nodes = nodes;
    for (int k = 0; k < N; ++k) {
        if (config_out) config_out[k] = ok ? leaf[k] : -1;
        if (window_out) window_out[k] = ok ? 0 : -1;
    }
    if (!ok) {
        res->index = ~0ull;
        res->cost = HUGE_VAL;
        res->max_latency_us = -1;
        return SMILESS_INFEASIBLE;
    }
    res->index = index_of(leaf);
    res->cost = cost[0];
    res->max_latency_us = lat[0];
    return SMILESS_OK;
}

int smiless_autoscale(const smiless_ctx *ctx, const double *slope_us, const double *intercept_us,
                      const int64_t *invocations, int64_t it_us, const int64_t *target_us,
                      smiless_autoscale_result *out) {
    if (!ctx || !slope_us || !intercept_us || !invocations || !target_us || !out) return SMILESS_EINVAL;
    if (!ctx->dag_loaded || !ctx->prof_loaded) return SMILESS_ESTATE;
    if (it_us < 0) return SMILESS_EINVAL;
    for (int k = 0; k < ctx->N; ++k) {
        smiless_autoscale_result best{-1, 0, 0, HUGE_VAL};
        const i64 G = invocations[k];
        if (G <= 0) {
            out[k] = smiless_autoscale_result{-1, 0, 0, 0.0};
            continue;
        }
        for (int c = 0; c < ctx->M[k]; ++c) {
            const int row = ctx->row0[k] + c;
            const double a = slope_us[row], b = intercept_us[row], lim = (double)target_us[k];
            auto ok = [&](i64 B) {
                volatile double prod = a * (double)B;   // two rounded operations, never an FMA
                return prod + b <= lim;
            };
            if (!ok(1)) continue;
            i64 lo = 1, hi = G;                           // bisection: largest feasible B
            while (lo < hi) {
                const i64 mid = lo + (hi - lo + 1) / 2;
                if (ok(mid)) lo = mid;
                else hi = mid - 1;
            }
            const i64 inst = (G + lo - 1) / lo;
            volatile double inst_it = (double)inst * (double)it_us;
            const double cost = inst_it * ctx->U[row];
            if (cost < best.cost) best = smiless_autoscale_result{c, lo, inst, cost};
        }
        out[k] = best;
    }
    return SMILESS_OK;
}

int smiless_autoscale_rows(const smiless_ctx *ctx, const double *slope_us, const double *intercept_us,
                           const int64_t *invocations, const int64_t *target_us, int64_t *batch_out,
                           int64_t *instances_out) {
    if (!ctx || !slope_us || !intercept_us || !invocations || !target_us || !batch_out || !instances_out)
        return SMILESS_EINVAL;
    if (!ctx->dag_loaded || !ctx->prof_loaded) return SMILESS_ESTATE;
    for (int k = 0; k < ctx->N; ++k) {
        const i64 G = invocations[k];
        for (int c = 0; c < ctx->M[k]; ++c) {
            const int row = ctx->row0[k] + c;
            const double sl = slope_us[row], ic = intercept_us[row], lim = (double)target_us[k];
            auto ok = [&](i64 B) {
                volatile double prod = sl * (double)B;   // two rounded operations, never an FMA
                return prod + ic <= lim;
            };
            batch_out[row] = 0;
            instances_out[row] = 0;
            if (G <= 0 || !ok(1)) continue;
            i64 lo = 1, hi = G;                            // bisection: largest feasible B
            while (lo < hi) {
                const i64 mid = lo + (hi - lo + 1) / 2;
                if (ok(mid)) lo = mid;
                else hi = mid - 1;
            }
            batch_out[row] = lo;
            instances_out[row] = (G + lo - 1) / lo;
        }
    }
    return SMILESS_OK;
}

int smiless_decompose_search(smiless_ctx *ctx, const smiless_plan_args *a, int64_t it_us, smiless_plan_result *res,
                             int32_t *config_out, int32_t *window_out, int64_t *n_paths) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!a || !res) return fail(ctx, SMILESS_EINVAL, "args / res is NULL");
    if (!a->row_windows_us) return fail(ctx, SMILESS_EINVAL, "decompose search needs row_windows_us (n_windows == 1)");
    if (a->n_fixed != 0) return fail(ctx, SMILESS_EINVAL, "decompose search does not take pinned digits");
    int rc = validate_args(ctx, a, true);
    if (rc) return rc;
    const int N = ctx->N;
    // successors and source -> sink paths (DFS)
    std::vector<std::vector<int>> succ(N);
    for (int k = 0; k < N; ++k)
        for (int e = ctx->pred_ptr[k]; e < ctx->pred_ptr[k + 1]; ++e) succ[ctx->pred_idx[e]].push_back(k);
    std::vector<std::vector<int>> paths;
    std::vector<int> cur;
    bool too_many = false;
    std::function<void(int)> walk = [&](int k) {
        if (too_many) return;
        cur.push_back(k);
        if (succ[k].empty()) {
            paths.push_back(cur);
            if (paths.size() > 4096) too_many = true;
        }
        for (int s_ : succ[k]) walk(s_);
        cur.pop_back();
    };
    for (int k = 0; k < N; ++k)
        if (ctx->pred_ptr[k] == ctx->pred_ptr[k + 1]) walk(k);
    if (too_many) return fail(ctx, SMILESS_EINVAL, "more than 4096 source-to-sink paths");
    // per-function cost ranking (Eq. 5 / Case II) and fastest config
    auto per_inv_cost = [&](int k, int m) {
        const int row = ctx->row0[k] + m;
        const i64 t = ctx->T[row], i = ctx->I[row];
        return ctx->U[row] * ((t + i < it_us) ? (double)(t + i) : (double)it_us);
    };
    auto I_of = [&](int k, int m) { return (i64)ctx->I[ctx->row0[k] + m]; };
    std::vector<std::vector<int>> rank(N);
    std::vector<int> fastest(N);
    for (int k = 0; k < N; ++k) {
        std::vector<int> o(ctx->M[k]);
        for (int m = 0; m < ctx->M[k]; ++m) o[m] = m;
        std::stable_sort(o.begin(), o.end(), [&](int x, int y) { return per_inv_cost(k, x) < per_inv_cost(k, y); });
        rank[k] = o;
        int f = 0;
        for (int m = 1; m < ctx->M[k]; ++m)
            if (I_of(k, m) < I_of(k, f)) f = m;
        fastest[k] = f;
    }
    const i64 sla = a->sla_us;
    // Top-1 per path with the closed-form latency sum(I)
    std::vector<std::vector<int>> choice(paths.size());
    for (size_t pi = 0; pi < paths.size(); ++pi) {
        const auto &P = paths[pi];
        const size_t L = P.size();
        std::vector<int> c(L);
        i64 lat = 0;
        for (size_t q = 0; q < L; ++q) { c[q] = rank[P[q]][0]; lat += I_of(P[q], c[q]); }
        if (lat > sla) {
            std::vector<int> chosen;
            for (size_t q = 0; q < L; ++q) {
                int pick = fastest[P[q]];
                for (int r = (q == 0 ? 1 : 0); r < ctx->M[P[q]]; ++r) {
                    i64 l = 0;
                    for (size_t z = 0; z < L; ++z)
                        l += I_of(P[z], z < q ? chosen[z] : (z == q ? rank[P[q]][r] : fastest[P[z]]));
                    if (l <= sla) { pick = rank[P[q]][r]; break; }
                }
                chosen.push_back(pick);
            }
            c = chosen;
        }
        choice[pi] = c;
    }
    // combine: shared functions take the fastest of the paths' choices ...
    std::vector<int> cfg(N, -1), n_on(N, 0);
    std::vector<i64> path_lat(paths.size(), 0);
    for (size_t pi = 0; pi < paths.size(); ++pi)
        for (size_t q = 0; q < paths[pi].size(); ++q) {
            const int k = paths[pi][q], m = choice[pi][q];
            path_lat[pi] += I_of(k, m);
            n_on[k] += 1;
            if (cfg[k] < 0 || I_of(k, m) < I_of(k, cfg[k])) cfg[k] = m;
        }
    // ... and functions on a single path move to their cheapest config that keeps that path's
    // closed-form latency at or below its latency before combining
    for (size_t pi = 0; pi < paths.size(); ++pi) {
        const auto &P = paths[pi];
        for (size_t q = 0; q < P.size(); ++q) {
            const int k = P[q];
            if (n_on[k] != 1) continue;
            i64 others = 0;
            for (size_t z = 0; z < P.size(); ++z)
                if (z != q) others += I_of(P[z], cfg[P[z]]);
            for (int r = 0; r < ctx->M[k]; ++r)
                if (others + I_of(k, rank[k][r]) <= path_lat[pi]) { cfg[k] = rank[k][r]; break; }
        }
    }
    // evaluate the combined plan with model M on the GPU
    u64 idx = 0;
    for (int k = 0; k < N; ++k) idx = idx * (u64)ctx->M[k] + (u64)cfg[k];
    double cost = 0.0;
    int64_t lat = 0;
    uint8_t ok = 0;
    if ((rc = smiless_evaluate(ctx, a, (const uint64_t *)&idx, 1, &cost, &lat, &ok))) return rc;
    memset(res, 0, sizeof *res);
    res->n_decided = res->n_full_evals = 1;
    if (n_paths) *n_paths = (int64_t)paths.size();
    for (int k = 0; k < N; ++k) {
        if (config_out) config_out[k] = ok ? cfg[k] : -1;
        if (window_out) window_out[k] = ok ? 0 : -1;
    }
    if (!ok) {
        res->index = ~0ull;
        res->cost = HUGE_VAL;
        res->max_latency_us = -1;
        return SMILESS_INFEASIBLE;
    }
    res->index = idx;
    res->cost = cost;
    res->max_latency_us = lat;
    return SMILESS_OK;
}

int smiless_decompose_plan_sharded(smiless_ctx *ctx, const smiless_plan_args *a, smiless_path_reduce_fn reduce,
                                   void *user, smiless_plan_result *res, int32_t *config_out, int32_t *window_out,
                                   int64_t *n_paths) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!a || !res) return fail(ctx, SMILESS_EINVAL, "args / res is NULL");
    if (a->n_fixed != 0) return fail(ctx, SMILESS_EINVAL, "decompose plan does not take pinned digits");
    if (a->row_windows_us) return fail(ctx, SMILESS_EINVAL, "decompose plan searches the window grid (no row windows)");
    // a space above 2^63 (C5) is evaluated with function 0's digit pinned: the index is then in
    // the suffix space of functions 1..N-1
    const int32_t digit0 = 0;
    smiless_plan_args av = *a;
    {
        u64 sp;
        if (ctx->dag_loaded && ctx->prof_loaded && a->n_windows >= 1 && a->n_windows <= SMILESS_MAX_WINDOWS &&
            !space_size_of(ctx, a->n_windows, 0, &sp)) {
            av.n_fixed = 1;
            av.fixed_digits = &digit0;
        }
    }
    int rc = validate_args(ctx, &av, true);
    if (rc) return rc;
    const int N = ctx->N, W = a->n_windows;
    // 1. decompose into source-to-sink paths (subgraphs with only sequential dependencies)
    std::vector<std::vector<int>> succ(N), paths;
    for (int k = 0; k < N; ++k)
        for (int e = ctx->pred_ptr[k]; e < ctx->pred_ptr[k + 1]; ++e) succ[ctx->pred_idx[e]].push_back(k);
    std::vector<int> cur;
    bool too_many = false;
    std::function<void(int)> walk = [&](int k) {
        if (too_many) return;
        cur.push_back(k);
        if (succ[k].empty()) {
            paths.push_back(cur);
            if (paths.size() > 4096) too_many = true;
        }
        for (int s_ : succ[k]) walk(s_);
        cur.pop_back();
    };
    for (int k = 0; k < N; ++k)
        if (ctx->pred_ptr[k] == ctx->pred_ptr[k + 1]) walk(k);
    if (too_many) return fail(ctx, SMILESS_EINVAL, "more than 4096 source-to-sink paths");
    // one child context per path length (a chain DAG): the NVRTC specialisation is shared by
    // every path of that length, its profiles are reloaded per path
    std::map<int, smiless_ctx *> subs;
    struct SubGuard {
        std::map<int, smiless_ctx *> &m;
        ~SubGuard() { for (auto &kv : m) smiless_destroy(kv.second); }
    } guard{subs};
    auto sub_for = [&](const std::vector<int> &P, smiless_ctx **out) -> int {
        const int L = (int)P.size();
        auto it = subs.find(L);
        if (it == subs.end()) {
            smiless_ctx *c = nullptr;
            int r = smiless_create(&c, ctx->device, ctx->stream);
            if (r) return fail(ctx, r, "decompose: cannot create a path context");
            it = subs.emplace(L, c).first;
        }
        smiless_ctx *c = it->second;
        std::vector<int32_t> ptr(L + 1), idx(std::max(L - 1, 1));
        ptr[0] = 0;
        for (int q = 0; q < L; ++q) {
            if (q > 0) idx[q - 1] = q - 1;
            ptr[q + 1] = q;                               // q has predecessor q - 1 (chain)
        }
        int r = smiless_load_dag(c, L, ptr.data(), idx.data());
        std::vector<int32_t> m, I, T;
        std::vector<double> U;
        for (int k : P) {
            m.push_back(ctx->M[k]);
            for (int cc = 0; cc < ctx->M[k]; ++cc) {
                I.push_back(ctx->I[ctx->row0[k] + cc]);
                T.push_back(ctx->T[ctx->row0[k] + cc]);
                U.push_back(ctx->U[ctx->row0[k] + cc]);
            }
        }
        if (!r) r = smiless_load_profiles(c, m.data(), I.data(), T.data(), U.data());
        if (r) return fail(ctx, r, "decompose: path context: %s", smiless_last_error(c));
        *out = c;
        return SMILESS_OK;
    };
    auto path_args = [&](const std::vector<int> &P, std::vector<int32_t> &inst) {
        smiless_plan_args pa = *a;
        pa.begin = pa.end = 0;
        pa.shard = 0;
        pa.n_shards = 0;
        pa.cost_out = nullptr;
        pa.cost_cap = 0.0;
        pa.flags = a->flags & (SMILESS_FLAG_ARRIVALS_ON_DEVICE | SMILESS_FLAG_FORCE_INT64);
        inst.clear();
        for (int k : P) inst.push_back(inst_of(a, k));
        pa.instances = inst.data();
        return pa;
    };
    // 2. each path's exhaustive optimum under model M (exact B&B plan of the chain on the GPU)
    std::vector<std::vector<int>> pc(paths.size()), pw(paths.size());
    std::vector<i64> plat(paths.size(), 0);
    std::vector<int32_t> inst;
    for (size_t pi = 0; pi < paths.size(); ++pi) {
        const auto &P = paths[pi];
        smiless_ctx *c = nullptr;
        if ((rc = sub_for(P, &c))) return rc;
        smiless_plan_args pa = path_args(P, inst);
        if (reduce) {                                    // this rank's interleaved share of the path
            pa.shard = a->shard;
            pa.n_shards = a->n_shards;
        }
        smiless_plan_result pr;
        std::vector<int32_t> co(P.size()), wo(P.size());
        rc = smiless_plan(c, &pa, &pr, co.data(), wo.data());
        if (rc < 0) return fail(ctx, rc, "decompose: path plan: %s", smiless_last_error(c));
        if (reduce) {
            // the caller reduces the ranks' path winners (its collective) into pr
            const int rr = reduce(user, (int32_t)pi, &pr);
            if (rr) return fail(ctx, SMILESS_EINVAL, "decompose: path reduce callback returned %d", rr);
            rc = pr.index == ~0ull ? SMILESS_INFEASIBLE : SMILESS_OK;
            if (rc == SMILESS_OK) {
                pa.shard = 0;
                pa.n_shards = 0;
                const int dr = smiless_decode(c, W, pr.index, &pa, co.data(), wo.data());
                if (dr) return fail(ctx, dr, "decompose: reduced path winner %llu does not decode",
                                    (unsigned long long)pr.index);
            }
        }
        if (rc == SMILESS_INFEASIBLE) {                  // no plan meets the SLA on this path alone
            memset(res, 0, sizeof *res);
            res->index = ~0ull;
            res->cost = HUGE_VAL;
            res->max_latency_us = -1;
            for (int k = 0; k < N; ++k) {
                if (config_out) config_out[k] = -1;
                if (window_out) window_out[k] = -1;
            }
            if (n_paths) *n_paths = (int64_t)paths.size();
            return SMILESS_INFEASIBLE;
        }
        pc[pi].assign(co.begin(), co.end());
        pw[pi].assign(wo.begin(), wo.end());
        plat[pi] = pr.max_latency_us;
    }
    // 3. combine (reading G25): a function on several paths takes the choice with the
    // shortest inference time among them (the rule for F_s / F_e of a parallel substructure) ...
    std::vector<int> cfg(N, -1), win(N, -1), n_on(N, 0);
    for (size_t pi = 0; pi < paths.size(); ++pi)
        for (size_t q = 0; q < paths[pi].size(); ++q) {
            const int k = paths[pi][q], m = pc[pi][q];
            n_on[k] += 1;
            if (cfg[k] < 0 || ctx->I[ctx->row0[k] + m] < ctx->I[ctx->row0[k] + cfg[k]]) {
                cfg[k] = m;
                win[k] = pw[pi][q];
            }
        }
    // ... and every function on one path only moves to its cheapest (configuration, window) that
    // keeps that path's model-M latency at or below its latency before combining (evaluated on
    // the GPU, one batch per function; ties to the lowest digit)
    for (size_t pi = 0; pi < paths.size(); ++pi) {
        const auto &P = paths[pi];
        smiless_ctx *c = nullptr;
        if ((rc = sub_for(P, &c))) return rc;
        smiless_plan_args pa = path_args(P, inst);         // (every rank evaluates these itself)
        for (size_t q = 0; q < P.size(); ++q) {
            const int k = P[q];
            if (n_on[k] != 1) continue;
            const int R = ctx->M[k] * W;
            std::vector<uint64_t> idx(R);
            for (int d = 0; d < R; ++d) {
                u64 v = 0;
                for (size_t z = 0; z < P.size(); ++z) {
                    const u64 dz = (z == q) ? (u64)d : (u64)cfg[P[z]] * (u64)W + (u64)win[P[z]];
                    v = v * ((u64)ctx->M[P[z]] * (u64)W) + dz;
                }
                idx[d] = v;
            }
            std::vector<double> cost(R);
            std::vector<int64_t> lat(R);
            std::vector<uint8_t> ok(R);
            rc = smiless_evaluate(c, &pa, idx.data(), R, cost.data(), lat.data(), ok.data());
            if (rc) return fail(ctx, rc, "decompose: path evaluate: %s", smiless_last_error(c));
            int best = -1;
            for (int d = 0; d < R; ++d)
                if (lat[d] <= plat[pi] && (best < 0 || cost[d] < cost[best])) best = d;
            if (best >= 0) {
                cfg[k] = best / W;
                win[k] = best % W;
            }
        }
    }
    // 4. the combined plan under model M on the whole DAG
    const int32_t d0 = cfg[0] * W + win[0];
    if (av.n_fixed == 1) av.fixed_digits = &d0;
    u64 idx = 0;
    for (int k = av.n_fixed; k < N; ++k) idx = idx * ((u64)ctx->M[k] * (u64)W) + (u64)cfg[k] * (u64)W + (u64)win[k];
    double cost = 0.0;
    int64_t lat = 0;
    uint8_t ok = 0;
    if ((rc = smiless_evaluate(ctx, &av, (const uint64_t *)&idx, 1, &cost, &lat, &ok))) return rc;
    memset(res, 0, sizeof *res);
    res->n_decided = res->n_full_evals = 1;
    if (n_paths) *n_paths = (int64_t)paths.size();
    for (int k = 0; k < N; ++k) {
        if (config_out) config_out[k] = ok ? cfg[k] : -1;
        if (window_out) window_out[k] = ok ? win[k] : -1;
    }
    if (!ok) {
        res->index = ~0ull;
        res->cost = HUGE_VAL;
        res->max_latency_us = -1;
        return SMILESS_INFEASIBLE;
    }
    res->index = idx;
    res->cost = cost;
    res->max_latency_us = lat;
    return SMILESS_OK;
}

int smiless_decompose_plan(smiless_ctx *ctx, const smiless_plan_args *a, smiless_plan_result *res,
                           int32_t *config_out, int32_t *window_out, int64_t *n_paths) {
    return smiless_decompose_plan_sharded(ctx, a, nullptr, nullptr, res, config_out, window_out, n_paths);
}

int smiless_plan_sla_sweep(smiless_ctx *ctx, const smiless_plan_args *a, const int64_t *slas, int32_t n_sla,
                           smiless_plan_result *res, int32_t *config_out, int32_t *window_out) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    if (!res || !slas) return fail(ctx, SMILESS_EINVAL, "res / slas is NULL");
    if (n_sla < 1 || n_sla > SMILESS_MAX_SLAS) return fail(ctx, SMILESS_EINVAL, "n_sla must be in [1, %d]", SMILESS_MAX_SLAS);
    if (a && a->cost_out) return fail(ctx, SMILESS_EINVAL, "cost_out is not supported by the SLA sweep");
    const int rc = plan_impl(ctx, a, (const i64 *)slas, n_sla, res, config_out, window_out);
    return rc < 0 ? rc : SMILESS_OK;
}

// ---- introspection (build checks, SASS inspection, tests) ---------------------------------
int smiless_kernel_source(smiless_ctx *ctx, const smiless_plan_args *a, char *buf, size_t cap, size_t *len) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    int rc = validate_args(ctx, a, false);
    if (rc) return rc;
    const RangePlan rp = range_plan(ctx, a);
    const i64 n_steps = a->n_arrivals - 1;
    const i64 n_off = std::max<i64>(4, (n_steps + rp.K - 1) / rp.K * rp.K);
    const bool off_smem = smem_bytes(ctx, a, rp, n_off, true) <= 227 * 1024;
    std::string s = full_source(ctx, a, rp, off_smem, 1);
    if (len) *len = s.size() + 1;
    if (buf && cap) {
        const size_t n = std::min(cap - 1, s.size());
        memcpy(buf, s.data(), n);
        buf[n] = '\0';
    }
    return SMILESS_OK;
}

int smiless_jit_compile(smiless_ctx *ctx, const smiless_plan_args *a, char *log, size_t logcap, void *cubin_out,
                        size_t cubin_cap, size_t *cubin_size) {
    if (!ctx) return SMILESS_EINVAL;
    ctx->err.clear();
    int rc = validate_args(ctx, a, false);
    if (rc) return rc;
    const RangePlan rp = range_plan(ctx, a);
    const i64 n_steps = a->n_arrivals - 1;
    const i64 n_off = std::max<i64>(4, (n_steps + rp.K - 1) / rp.K * rp.K);
    const bool off_smem = smem_bytes(ctx, a, rp, n_off, true) <= 227 * 1024;
    std::vector<char> cubin;
    std::string lg;
    rc = nvrtc_compile(ctx, full_source(ctx, a, rp, off_smem, min_blocks()), cubin, lg);
    if (log && logcap) {
        const size_t n = std::min(logcap - 1, lg.size());
        memcpy(log, lg.data(), n);
        log[n] = '\0';
    }
    if (cubin_size) *cubin_size = cubin.size();
    if (cubin_out && cubin_cap >= cubin.size()) memcpy(cubin_out, cubin.data(), cubin.size());
    return rc;
}

}  // extern "C"
