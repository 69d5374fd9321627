// kernels.cu -- DAG-independent kernels of the hot path (compiled by nvcc for sm_100a):
//   * prep_offsets: validate arrivals, clamp gaps at d_cap, write
//                     chunk-relative offsets for the evaluator, R = r_{J-1} - r_0
//   * reduce_best    (a8): fold per-CTA (cost bits, index) slots into the winner
//   * eval_exact     (a6/a7 exact, B9): int64 absolute-time evaluation of explicit
//                     candidate indices, no pruning, no clamping (smiless_evaluate and
//                     the winner re-evaluation of smiless_plan, a10)
// The DAG-specialised evaluator lives in evaluator.cuh (NVRTC).
#include <cstdint>
#include <cuda_runtime.h>

#include "kernels.h"

typedef long long i64;
typedef unsigned long long u64;

namespace smiless_dev {

// One thread per chunk of K steps; step s (0-based) is arrival j = s + 1.
// off[s] = sum_{i = chunk start}^{s} min(r_{i+1} - r_i, d_cap), i.e. the clamped arrival
// time of j = s + 1 relative to the chunk base (the arrival just before the chunk).
// rrem[q] = r_{J-1} - r_{(q+1)K}: the real (unclamped) time left after chunk q, used by the
// evaluator's cost bound (0 past the last full chunk).
template <typename T>
__global__ void prep_offsets_kernel(const i64 *__restrict__ arr, i64 J, i64 d_cap, int K, T *__restrict__ off,
                                    i64 n_off, i64 *__restrict__ scal, int *__restrict__ err, i64 *__restrict__ rrem) {
    const i64 n_steps = J - 1;
    const i64 q = (i64)blockIdx.x * blockDim.x + threadIdx.x;
    const i64 s0 = q * K;
    if (s0 >= n_off) return;
    rrem[q] = (q + 1) * K <= n_steps ? arr[J - 1] - arr[(q + 1) * K] : 0;
    i64 acc = 0;
    const i64 LIM = (i64)1 << 62;
    for (i64 s = s0; s < s0 + K && s < n_off; ++s) {
        if (s < n_steps) {
            const i64 a = arr[s], b = arr[s + 1];
            if (a <= -LIM || a >= LIM || b <= -LIM || b >= LIM) atomicOr(err, 2);
            const i64 gap = b - a;
            if (gap < 0) atomicOr(err, 1);
            acc += gap < d_cap ? gap : d_cap;
            off[s] = (T)acc;
            if (s == n_steps - 1) scal[1] = acc;
        } else {
            off[s] = (T)0;
        }
    }
    if (q == 0) {
        const i64 a = arr[0], b = arr[J - 1];
        if (a <= -LIM || a >= LIM || b <= -LIM || b >= LIM) atomicOr(err, 2);
        scal[0] = b - a;
        if (n_steps == 0) scal[1] = 0;
    }
}

// Scale-out plans (NEXT-4): scal[2 + (n-1)] = sum_{i < min(n, J)} (r_{J-1-i} - r_i) for
// n = 1..16 (real time), scal[18 + i] = clamped offset of arrival J-1-i in the evaluator's final
// frame (the base of the last chunk it runs: arrival K * q_last), i = 0..15.  One thread.
__global__ void prep_tail_kernel(const i64 *__restrict__ arr, i64 J, i64 d_cap, int K, i64 *__restrict__ scal) {
    if (blockIdx.x != 0 || threadIdx.x != 0) return;
    const i64 n_steps = J - 1, nfc = n_steps / K;
    const i64 q_last = nfc == 0 ? 0 : (nfc * K < n_steps ? nfc : nfc - 1);
    const i64 jb = (i64)K * q_last;
    i64 acc = 0;
    for (int n = 1; n <= 16; ++n) {
        const i64 i = n - 1;
        if (i < J) acc += arr[J - 1 - i] - arr[i];
        scal[2 + i] = acc;
    }
    for (int i = 0; i < 16; ++i) {
        const i64 j = J - 1 - i;
        i64 o = 0;
        if (j >= jb) {
            for (i64 m = jb; m < j; ++m) { const i64 g = arr[m + 1] - arr[m]; o += g < d_cap ? g : d_cap; }
        } else if (j >= 0) {
            for (i64 m = j; m < jb; ++m) { const i64 g = arr[m + 1] - arr[m]; o -= g < d_cap ? g : d_cap; }
        }
        scal[18 + i] = o;
    }
    // per instance count n = 1..16 and instance i < n (requests i, i + n, ...): the real span
    // R_i = r_{last_i} - r_i at scal[34 + (n-1)*16 + i] and the request count c_i at
    // scal[290 + (n-1)*16 + i] (0 when i >= J): the static cost bound of a scale-out function
    for (int n = 1; n <= 16; ++n)
        for (int i = 0; i < 16; ++i) {
            i64 span = 0, cnt = 0;
            if (i < n && i < J) {
                cnt = (J - 1 - i) / n + 1;
                span = arr[i + (cnt - 1) * n] - arr[i];
            }
            scal[34 + (n - 1) * 16 + i] = span;
            scal[290 + (n - 1) * 16 + i] = cnt;
        }
}

__device__ __forceinline__ bool key_less(u64 ca, u64 ia, u64 cb, u64 ib) {
    return ca < cb || (ca == cb && ia < ib);
}

__global__ void reduce_best_kernel(const u64 *__restrict__ slots, int n, int stride, ResBlock *__restrict__ res) {
    __shared__ u64 sc[256], si[256];
    u64 c = ~0ull, i = ~0ull;
    for (int b = threadIdx.x; b < n; b += blockDim.x) {
        const u64 *sl = slots + 2 * (size_t)b * stride;
        if (key_less(sl[0], sl[1], c, i)) { c = sl[0]; i = sl[1]; }
    }
    sc[threadIdx.x] = c;
    si[threadIdx.x] = i;
    __syncthreads();
    for (int s = blockDim.x / 2; s > 0; s >>= 1) {
        if (threadIdx.x < s && key_less(sc[threadIdx.x + s], si[threadIdx.x + s], sc[threadIdx.x], si[threadIdx.x])) {
            sc[threadIdx.x] = sc[threadIdx.x + s];
            si[threadIdx.x] = si[threadIdx.x + s];
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        res->best_c = sc[0];
        res->best_i = si[0];
    }
}

// Exact evaluation, absolute int64 times, generic DAG (runtime CSR in device memory), the
// plain case split of model M (with scale-out instances, reading G26: request j
// on instance j mod n_k, previous completion D[k][j - n_k]) with per-step billing -- independent of the
// NVRTC evaluator's reformulations.  One WARP per candidate, lane k = function k, run as a
// wavefront: a function's level is 1 + the highest level of its predecessors, and at
// iteration t lane k handles invocation j = t - level_k.  Its predecessors (lower levels)
// finished invocation j in earlier iterations and left D[p][j] in a per-warp shared ring of
// 32 invocations (level gaps are <= 31, so a slot is never overwritten before it is read);
// one __syncwarp per iteration orders the ring.  A whole invocation of the DAG thus costs
// one iteration of the warp instead of N dependent steps of one thread.
#define EXACT_WARPS 4

// arrivals staged per warp in a shared ring of 512 (4 blocks of 128), each block fetched with
// cp.async 256 invocations before it is read (the lanes read j in [it - 31, it])
#define EXACT_ARR_RING 512
#define EXACT_ARR_BLOCK 128

__device__ __forceinline__ void exact_fetch_block(long long *ring_arr, const long long *arr, i64 J, i64 b, int lane) {
    // block b = arrivals [b * 128, b * 128 + 128): 8-byte copies (any int64-aligned source), 4 per
    // lane; past J: nothing
    for (int q = lane; q < EXACT_ARR_BLOCK; q += 32) {
        const i64 j0 = b * EXACT_ARR_BLOCK + q;
        if (j0 < J) {
            const unsigned dst = (unsigned)__cvta_generic_to_shared(ring_arr + (j0 & (EXACT_ARR_RING - 1)));
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst), "l"(arr + j0) : "memory");
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

__global__ void __launch_bounds__(32 * EXACT_WARPS) eval_exact_kernel(ExactParams p) {
    __shared__ long long ring[EXACT_WARPS][SMILESS_DEV_MAX_FUNCS][32];   // [warp][function][j % 32]
    __shared__ __align__(16) long long ring_arr[EXACT_WARPS][EXACT_ARR_RING];
    const unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const i64 t = ((i64)blockIdx.x * blockDim.x + threadIdx.x) >> 5;   // candidate of this warp
    if (t >= p.n) return;                                                // warp-uniform
    ResBlock *res = p.idx_from_res ? p.res + t : nullptr;
    const i64 sla = p.idx_from_res ? p.slas[t] : p.sla;
    const u64 index = p.idx_from_res ? res->best_i : p.idx[t];
    if (index == ~0ull) {
        if (res && lane == 0) { res->feasible = 0; res->cost = 0.0; res->maxlat = -1; }
        return;
    }
    const int N = p.N, W = p.W;
    const bool act = lane < N;
    const int k = act ? lane : 0;
    // ---- decode this lane's digit: index = sum_k d_k S_k over functions n_fixed..N-1 --------
    int cfg = 0, win = 0;
    if (lane < p.n_fixed) {
        cfg = p.fixed[lane] / W;
        win = p.fixed[lane] % W;
    } else if (act) {
        u64 stride = 1;
        for (int q = N - 1; q > k; --q) stride *= (u64)p.M[q] * (u64)W;
        const u64 d = (index / stride) % ((u64)p.M[k] * (u64)W);
        cfg = (int)(d / (u64)W);
        win = (int)(d % (u64)W);
    }
    const int row = p.row0[k] + cfg;
    const i64 I = act ? p.tabI[row] : 0, T = act ? p.tabT[row] : 0;
    const i64 w = act ? (p.rowwin ? p.rowwin[row] : p.win[win]) : 0;
    const int nin = act ? p.inst[k] : 1;                // instances (request j on instance j mod nin)
    const int e0 = act ? p.pred_ptr[k] : 0, deg = act ? p.pred_ptr[k + 1] - e0 : 0;
    const bool sink = act && ((p.sinkmask >> k) & 1u);
    int pc[8];                                            // first predecessors, in registers
#pragma unroll
    for (int e = 0; e < 8; ++e) pc[e] = e < deg ? p.pred_idx[e0 + e] : 0;
    int maxdeg = deg;
#pragma unroll
    for (int m = 16; m > 0; m >>= 1) maxdeg = max(maxdeg, __shfl_xor_sync(FULL, maxdeg, m));
    // ---- topological levels (Bellman-Ford over the warp, N passes at most) -----------------
    int lvl = 0;
    for (int pass = 0; pass < N; ++pass) {
        int l2 = 0;
        for (int e = 0; e < maxdeg; ++e) {
            const int src = e < deg ? p.pred_idx[e0 + e] : lane;
            const int lp = __shfl_sync(FULL, lvl, src);
            if (e < deg) l2 = max(l2, lp + 1);
        }
        lvl = l2;
    }
    int nlev = act ? lvl + 1 : 1;
#pragma unroll
    for (int m = 16; m > 0; m >>= 1) nlev = max(nlev, __shfl_xor_sync(FULL, nlev, m));

    long long (*rg)[32] = ring[wib];
    const i64 J = p.J;
    i64 D = 0, billed = 0, maxlat = INT64_MIN;
    long long *ra = ring_arr[wib];
    // blocks 0, 1 now (waited for), block m + 2 at iteration 128 m (waited for 128 iterations later)
    exact_fetch_block(ra, p.arr, J, 0, lane);
    exact_fetch_block(ra, p.arr, J, 1, lane);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
    const i64 wT = w + T;                                 // per-lane constants of the case split
    const bool keep = w == 0;                             // keep-alive (Case II)
    const int n_it = (int)(J + nlev - 1);                 // J <= 2^31 (validated): 32-bit step counters
    const int Ji = (int)J;
    for (int it = 0; it < n_it; ++it) {
        if ((it & (EXACT_ARR_BLOCK - 1)) == 0) {
            // the previous fetch (block it / 128 + 1, read from the next block boundary on) has
            // landed once at most the newest group is pending; then fetch block it / 128 + 2
            asm volatile("cp.async.wait_group 0;" ::: "memory");
            __syncwarp();
            exact_fetch_block(ra, p.arr, J, it / EXACT_ARR_BLOCK + 2, lane);
        }
        const int j = it - lvl;
        const bool on = act && j >= 0 && j < Ji;
        const i64 r = on ? ra[j & (EXACT_ARR_RING - 1)] : 0;
        if (on) {
            i64 x = r;                                    // sources: the request's arrival
            const int sl = j & 31;
#pragma unroll
            for (int e = 0; e < 8; ++e) {                 // AND-join: max over predecessors
                if (e < deg) {
                    const i64 d = rg[pc[e]][sl];
                    x = e == 0 ? d : max(x, d);
                }
            }
            for (int e = 8; e < deg; ++e) x = max(x, rg[p.pred_idx[e0 + e]][sl]);
            // the case split of model M as selects (lanes of one warp take different cases;
            // straight-line code keeps them converged)
            // previous completion on this request's instance: D[k][j - nin] (own ring slot,
            // nin <= 16 < 32 so it is still there), or the register copy for one instance
            const i64 f = nin == 1 ? D : rg[k][(j - nin) & 31], g = x - f;
            // s = f + w: x < s <=> g < w, x < s + T <=> g < w + T (compared on g, no s formed)
            const bool busy = g <= 0;                     // busy: FIFO, stays warm (G6)
            const bool cold = g < w;                      // pre-warm not begun: cold (G3)
            const bool part = g < wT;                     // init partly covered (G4); else covered (Case I)
            i64 start = busy ? f : keep ? x : cold ? x + T : part ? f + wT : x;
            i64 bill = busy ? 0 : keep ? g : part ? T : g - w;
            if (j < nin) {                                // first invocation of an instance pre-warmed (G5)
                start = x;
                bill = T;
            }
            D = start + I;
            billed += bill + I;
            rg[k][j & 31] = D;
            if (sink) maxlat = max(maxlat, D - r);
        }
        __syncwarp();
    }
#pragma unroll
    for (int m = 16; m > 0; m >>= 1)
        maxlat = max(maxlat, (i64)__shfl_xor_sync(FULL, (unsigned long long)maxlat, m));
    // cost = ((U_0 E_0 + U_1 E_1) + ...) left to right, IEEE mul/add, no FMA (G15)
    const double term = act ? __dmul_rn(p.tabU[row], (double)billed) : 0.0;
    double cost = 0.0;
    for (int q = 0; q < N; ++q) {
        const double tq = __shfl_sync(FULL, term, q);
        cost = (q == 0) ? tq : __dadd_rn(cost, tq);
    }
    const unsigned char ok = maxlat <= sla ? 1 : 0;
    if (res) {
        if (act) { res->cfg[k] = cfg; res->win[k] = win; }
        if (lane == 0) { res->cost = cost; res->maxlat = maxlat; res->feasible = ok; }
    } else if (lane == 0) {
        p.cost[t] = cost;
        p.maxlat[t] = maxlat;
        p.feas[t] = ok;
    }
}

}  // namespace smiless_dev

extern "C" {

int smiless_dev_prep_offsets(const long long *arr, long long J, long long d_cap, int K, int time64, void *off,
                             long long n_off, long long *scal, int *err, long long *rrem, cudaStream_t st) {
    const long long n_threads = (n_off + K - 1) / K;
    const int bs = 128;
    const unsigned grid = (unsigned)((n_threads + bs - 1) / bs);
    if (grid == 0) return 0;
    if (time64)
        smiless_dev::prep_offsets_kernel<long long><<<grid, bs, 0, st>>>(arr, J, d_cap, K, (long long *)off, n_off, scal, err,
                                                                         rrem);
    else
        smiless_dev::prep_offsets_kernel<int><<<grid, bs, 0, st>>>(arr, J, d_cap, K, (int *)off, n_off, scal, err, rrem);
    return (int)cudaGetLastError();
}

int smiless_dev_prep_tail(const long long *arr, long long J, long long d_cap, int K, long long *scal, cudaStream_t st) {
    smiless_dev::prep_tail_kernel<<<1, 32, 0, st>>>(arr, J, d_cap, K, scal);
    return (int)cudaGetLastError();
}

int smiless_dev_reduce_best(const unsigned long long *slots, int n, int stride, ResBlock *res, cudaStream_t st) {
    smiless_dev::reduce_best_kernel<<<1, 256, 0, st>>>(slots, n, stride, res);
    return (int)cudaGetLastError();
}

int smiless_dev_eval_exact(const ExactParams *p, cudaStream_t st) {
    const int bs = 32 * EXACT_WARPS;                      // one candidate (warp) each
    const unsigned grid = (unsigned)((p->n * 32 + bs - 1) / bs);
    if (grid == 0) return 0;
    smiless_dev::eval_exact_kernel<<<grid, bs, 0, st>>>(*p);
    return (int)cudaGetLastError();
}

}  // extern "C"
