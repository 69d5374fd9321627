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
template <typename T>
__global__ void prep_offsets_kernel(const i64 *__restrict__ arr, i64 J, i64 d_cap, int K, T *__restrict__ off,
                                    i64 n_off, i64 *__restrict__ scal, int *__restrict__ err) {
    const i64 n_steps = J - 1;
    const i64 q = (i64)blockIdx.x * blockDim.x + threadIdx.x;
    const i64 s0 = q * K;
    if (s0 >= n_off) return;
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

// Exact evaluation, absolute int64 times, generic DAG (runtime CSR in device memory).
__global__ void eval_exact_kernel(ExactParams p) {
    const i64 t = (i64)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= p.n) return;
    ResBlock *res = p.idx_from_res ? p.res + t : nullptr;
    const i64 sla = p.idx_from_res ? p.slas[t] : p.sla;
    u64 index = p.idx_from_res ? res->best_i : p.idx[t];
    if (index == ~0ull) {
        if (res) { res->feasible = 0; res->cost = 0.0; res->maxlat = -1; }
        return;
    }
    const int N = p.N, W = p.W;
    int cfg[SMILESS_DEV_MAX_FUNCS], win[SMILESS_DEV_MAX_FUNCS];
    for (int k = N - 1; k >= p.n_fixed; --k) {
        const u64 radix = (u64)p.M[k] * (u64)W;
        const u64 d = index % radix;
        index /= radix;
        cfg[k] = (int)(d / (u64)W);
        win[k] = (int)(d % (u64)W);
    }
    for (int k = 0; k < p.n_fixed; ++k) {
        cfg[k] = p.fixed[k] / W;
        win[k] = p.fixed[k] % W;
    }
    i64 I[SMILESS_DEV_MAX_FUNCS], T[SMILESS_DEV_MAX_FUNCS], w[SMILESS_DEV_MAX_FUNCS];
    i64 D[SMILESS_DEV_MAX_FUNCS], billed[SMILESS_DEV_MAX_FUNCS];
    for (int k = 0; k < N; ++k) {
        const int row = p.row0[k] + cfg[k];
        I[k] = p.tabI[row];
        T[k] = p.tabT[row];
        w[k] = p.rowwin ? p.rowwin[row] : p.win[win[k]];
        billed[k] = 0;
        D[k] = 0;
    }
    i64 maxlat = INT64_MIN;
    for (i64 j = 0; j < p.J; ++j) {
        const i64 r = p.arr[j];
        i64 lat = INT64_MIN;
        for (int k = 0; k < N; ++k) {
            i64 x;
            const int e0 = p.pred_ptr[k], e1 = p.pred_ptr[k + 1];
            if (e0 == e1) {
                x = r;
            } else {
                x = D[p.pred_idx[e0]];
                for (int e = e0 + 1; e < e1; ++e) x = max(x, D[p.pred_idx[e]]);
            }
            i64 start, bill;
            if (j == 0) {
                start = x;
                bill = T[k];
            } else {
                const i64 f = D[k], g = x - f;
                if (g <= 0) {
                    start = f;
                    bill = 0;
                } else {
                    const i64 te = w[k] == 0 ? 0 : T[k];
                    const i64 u = min(g, w[k]);
                    start = f + max(u + te, g);
                    bill = max(te, g - w[k]);
                }
            }
            D[k] = start + I[k];
            billed[k] += bill + I[k];
            if ((p.sinkmask >> k) & 1u) lat = max(lat, D[k] - r);
        }
        maxlat = max(maxlat, lat);
    }
    double cost = 0.0;
    for (int k = 0; k < N; ++k) {
        const double term = __dmul_rn(p.tabU[p.row0[k] + cfg[k]], (double)billed[k]);
        cost = (k == 0) ? term : __dadd_rn(cost, term);
    }
    const unsigned char ok = maxlat <= sla ? 1 : 0;
    if (res) {
        res->cost = cost;
        res->maxlat = maxlat;
        res->feasible = ok;
        for (int k = 0; k < N; ++k) { res->cfg[k] = cfg[k]; res->win[k] = win[k]; }
    } else {
        p.cost[t] = cost;
        p.maxlat[t] = maxlat;
        p.feas[t] = ok;
    }
}

}  // namespace smiless_dev

extern "C" {

int smiless_dev_prep_offsets(const long long *arr, long long J, long long d_cap, int K, int time64, void *off,
                             long long n_off, long long *scal, int *err, cudaStream_t st) {
    const long long n_threads = (n_off + K - 1) / K;
    const int bs = 128;
    const unsigned grid = (unsigned)((n_threads + bs - 1) / bs);
    if (grid == 0) return 0;
    if (time64)
        smiless_dev::prep_offsets_kernel<long long><<<grid, bs, 0, st>>>(arr, J, d_cap, K, (long long *)off, n_off, scal, err);
    else
        smiless_dev::prep_offsets_kernel<int><<<grid, bs, 0, st>>>(arr, J, d_cap, K, (int *)off, n_off, scal, err);
    return (int)cudaGetLastError();
}

int smiless_dev_reduce_best(const unsigned long long *slots, int n, int stride, ResBlock *res, cudaStream_t st) {
    smiless_dev::reduce_best_kernel<<<1, 256, 0, st>>>(slots, n, stride, res);
    return (int)cudaGetLastError();
}

int smiless_dev_eval_exact(const ExactParams *p, cudaStream_t st) {
    const int bs = 128;
    const unsigned grid = (unsigned)((p->n + bs - 1) / bs);
    if (grid == 0) return 0;
    smiless_dev::eval_exact_kernel<<<grid, bs, 0, st>>>(*p);
    return (int)cudaGetLastError();
}

}  // extern "C"
