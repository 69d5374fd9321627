// kernels.h -- internal interface between host.cpp and kernels.cu (not part of the C ABI).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#define SMILESS_DEV_MAX_FUNCS 32
#define SMILESS_DEV_MAX_WINDOWS 32
#define SMILESS_DEV_MAX_EDGES 512

// Device-resident result of one smiless_plan call (copied back with one D2H).
struct ResBlock {
    unsigned long long best_c;   // cost bits of the winner (UINT64_MAX: none)
    unsigned long long best_i;   // winner index (suffix space)
    double cost;                 // exact re-evaluated cost
    long long maxlat;            // exact max latency
    int feasible;
    int err;                     // arrival validation flags (1: decreasing, 2: out of range)
    unsigned long long stats[2]; // decided, full evaluations
    int cfg[SMILESS_DEV_MAX_FUNCS];
    int win[SMILESS_DEV_MAX_FUNCS];
};

struct ExactParams {
    const int *tabI;
    const int *tabT;
    const double *tabU;
    const long long *arr;
    long long J;
    const unsigned long long *idx;
    long long n;
    double *cost;
    long long *maxlat;
    unsigned char *feas;
    ResBlock *res;               // when idx_from_res: thread t evaluates res[t].best_i with slas[t]
    int idx_from_res;
    long long sla;
    long long slas[8];
    int N, W, n_fixed;
    unsigned sinkmask;
    const int *pred_ptr;         // device [N+1]
    const int *pred_idx;         // device [E]
    int M[SMILESS_DEV_MAX_FUNCS];
    int row0[SMILESS_DEV_MAX_FUNCS];
    int win[SMILESS_DEV_MAX_WINDOWS];
    int fixed[SMILESS_DEV_MAX_FUNCS];
    const int *rowwin;           // per-row windows (NULL: the grid)
    int inst[SMILESS_DEV_MAX_FUNCS];   // scale-out instances per function (>= 1, <= 16)
};

extern "C" {
int smiless_dev_prep_offsets(const long long *arr, long long J, long long d_cap, int K, int time64, void *off,
                             long long n_off, long long *scal, int *err, long long *rrem, cudaStream_t st);
int smiless_dev_prep_tail(const long long *arr, long long J, long long d_cap, int K, long long *scal, cudaStream_t st);
int smiless_dev_reduce_best(const unsigned long long *slots, int n, int stride, ResBlock *res, cudaStream_t st);
int smiless_dev_eval_exact(const ExactParams *p, cudaStream_t st);
}
