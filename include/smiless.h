/*
 * smiless.h -- C ABI of the B200-native SMIless co-optimisation hot path.
 *
 * The operation (PAPER.md line citations, "P:n"):
 *
 *   Given an application DAG of N serverless inference functions,
 *   per-function x per-configuration profiles -- inference time I, init time T
 *   (T = mu + 3 sigma) and unit price U (Eq. (3)) --,
 *   a cold-start policy set S = a grid of pre-warming windows (window 0
 *   = keep alive), a predicted invocation-arrival sequence
 *   and an SLA on end-to-end latency (Eq. (4), default 2 s P:283),
 *   return the exhaustive optimum ("OPT ... determined through
 *   exhaustive search") of
 *
 *       min_{chi, phi}  sum_k C_k(*_k, /\_k) = sum_k E_k * U(*_k)   (Eq. 3, 4)
 *       s.t.            L(chi, phi) <= SLA      for every request
 *
 *   where each candidate (config *_k and window /\_k for every function) is
 *   simulated over the whole arrival sequence with model M (DESIGN.md "Model
 *   M": the Case I / II / III rules of P:169-200 applied per invocation; the
 *   E2E latency is "sum along sequential stages, max over parallel branches"
 *   with FIFO waiting and cold-start penalties; E_k = init + inference +
 *   loaded-idle time).  Ties on cost go to the LOWEST candidate index.
 *
 * Units: all times are integer microseconds, prices are double per
 * microsecond.  Candidate index order (mixed radix): function n_fixed is the
 * most significant digit, function N-1 the least; digit d_k = c_k * W + w_k
 * (config major, window minor); radix of function k is M_k * W.
 *
 * Ownership: the caller owns every buffer; inputs are copied before the call
 * returns and no pointer is retained; outputs are written only when the call
 * returns SMILESS_OK or SMILESS_INFEASIBLE.  The CUDA stream is borrowed.
 * Threading: one context per host thread.  Every call is synchronous with
 * respect to the host (results are on the host when it returns).
 *
 * Errors: negative return codes; smiless_last_error() returns a message.
 * There is no CPU fallback: a missing GPU, driver or NVRTC returns
 * SMILESS_ECUDA / SMILESS_EJIT.
 */
#ifndef SMILESS_H
#define SMILESS_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define SMILESS_API __attribute__((visibility("default")))
#else
#define SMILESS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct smiless_ctx smiless_ctx;

enum {
    SMILESS_OK = 0,          /* success                                               */
    SMILESS_INFEASIBLE = 1,  /* success, but no candidate meets the SLA (reading G13)  */
    SMILESS_EINVAL = -1,     /* bad argument (null, size, range, unsorted arrivals ...) */
    SMILESS_ENOTTOPO = -2,   /* DAG not a topologically ordered predecessor CSR         */
    SMILESS_ERANGE = -3,     /* candidate space exceeds 2^63 (indices must fit int64)   */
    SMILESS_ESTATE = -4,     /* call order: plan/evaluate before load_dag+load_profiles */
    SMILESS_ECUDA = -5,      /* CUDA runtime/driver failure or no device                */
    SMILESS_ENOMEM = -6,     /* host or device allocation failed                        */
    SMILESS_EJIT = -7        /* NVRTC specialisation of the evaluator failed            */
};

/* smiless_plan_args.flags */
enum {
    SMILESS_FLAG_NO_PRUNE = 1u,            /* throughput mode: walk every candidate to j = J-1 */
    SMILESS_FLAG_ARRIVALS_ON_DEVICE = 2u,  /* arrivals_us is a device pointer (HBM-resident)   */
    SMILESS_FLAG_FORCE_INT64 = 4u,         /* use the int64 evaluator even if int32 is exact   */
    SMILESS_FLAG_COST_CAP = 8u             /* only candidates with cost <= cost_cap are eligible
                                              (prune mode, smiless_plan only)                  */
};

#define SMILESS_MAX_FUNCS 32
#define SMILESS_MAX_WINDOWS 32
#define SMILESS_MAX_CONFIGS 256
#define SMILESS_MAX_SLAS 8
#define SMILESS_MAX_INSTANCES 16

/* Create a context bound to CUDA device `cuda_device` and stream `cuda_stream`
 * (a cudaStream_t; NULL = the legacy default stream; borrowed, not owned).
 * Host-only calls (load_*, space_size, decode) never touch the GPU; device
 * resources are acquired on the first plan/evaluate call.
 * Returns OK, EINVAL (out == NULL or device < 0) or ENOMEM. */
SMILESS_API int smiless_create(smiless_ctx **out, int cuda_device, void *cuda_stream);

/* Replace the borrowed stream used by later calls. */
SMILESS_API int smiless_set_stream(smiless_ctx *ctx, void *cuda_stream);

/* Release everything the context owns.  NULL-safe. */
SMILESS_API void smiless_destroy(smiless_ctx *ctx);

/* Message of the last failing call on ctx ("" if none).  Owned by ctx; valid
 * until the next call on ctx.  ctx == NULL gives the message of the last
 * failed smiless_create on this thread. */
SMILESS_API const char *smiless_last_error(const smiless_ctx *ctx);

/* Load the application DAG (NetworkX in the paper)
 * as a topologically ordered CSR over PREDECESSORS: function k's predecessors
 * are pred_idx[pred_ptr[k] .. pred_ptr[k+1]), each p < k, no duplicates.
 * Sources = empty predecessor list (they receive the request);
 * sinks = functions no one lists (the request completes when all sinks have).
 * 1 <= n_funcs <= SMILESS_MAX_FUNCS; pred_ptr has n_funcs+1 entries,
 * pred_ptr[0] == 0, non-decreasing; pred_idx may be NULL when it is empty.
 * Returns OK, EINVAL or ENOTTOPO.  Invalidates loaded profiles' compiled state. */
SMILESS_API int smiless_load_dag(smiless_ctx *ctx, int32_t n_funcs, const int32_t *pred_ptr, const int32_t *pred_idx);

/* Load per-function x per-config profiles: function k has
 * n_configs[k] (1..SMILESS_MAX_CONFIGS) rows; exec_us, init_us and
 * price_per_us are function-major, config-minor, length sum(n_configs).
 * 0 <= exec_us, init_us < 2^29; price_per_us finite and >= 0.
 * Requires a loaded DAG (else ESTATE).  Returns OK, EINVAL or ESTATE. */
SMILESS_API int smiless_load_profiles(smiless_ctx *ctx, const int32_t *n_configs, const int32_t *exec_us,
                          const int32_t *init_us, const double *price_per_us);

typedef struct {
    const int64_t *arrivals_us;   /* [n_arrivals] predicted arrivals r_0 <= r_1 <= ...;
                                     host pointer, or device pointer with FLAG_ARRIVALS_ON_DEVICE;
                                     |r_j| < 2^62                                                    */
    int64_t n_arrivals;           /* J >= 1                                                         */
    int64_t sla_us;               /* 0 <= SLA < 2^29; feasible iff max_j L_j <= SLA (G8)      */
    const int32_t *windows_us;    /* [n_windows] strictly increasing, 0 <= w < 2^29 (0 = keep-alive) */
    int32_t n_windows;            /* 1 <= W <= SMILESS_MAX_WINDOWS                                   */
    int32_t n_fixed;              /* digits of functions 0..n_fixed-1 are pinned (0 <= n_fixed <= N) */
    const int32_t *fixed_digits;  /* [n_fixed] digit = config * W + window; NULL if n_fixed == 0      */
    uint64_t begin, end;          /* index sub-range [begin, end) of the suffix space; end = 0: all  */
    uint32_t flags;               /* SMILESS_FLAG_*                                                  */
    int32_t shard, n_shards;      /* multi-GPU: this rank plans chunks c with c % n_shards == shard;
                                     n_shards = 0 or 1: everything                                   */
    double *cost_out;             /* optional (testing): host array [end - begin] receiving every
                                     candidate's cost as the evaluator computed it, NaN when it is
                                     infeasible or was pruned; NULL = off; end - begin <= 2^26     */
    const int32_t *row_windows_us;/* optional [sum(n_configs)] host array: the pre-warm window of
                                     each (function, config) row instead of a searched grid (the
                                     paper's adaptive pre-warming; see
                                     smiless_derive_windows); requires n_windows == 1 (windows_us
                                     is then ignored); 0 <= w < 2^29                               */
    double cost_cap;              /* with SMILESS_FLAG_COST_CAP: the plan is the argmin over the
                                     feasible candidates whose cost is <= cost_cap (INFEASIBLE if
                                     none), so a cap >= OPT returns OPT exactly.  Passing the cost of
                                     a plan known to be feasible (a heuristic's, the previous
                                     re-plan's) lets the evaluator's cost bound prune from the first
                                     launch (DESIGN.md section 5 item 11).  cost_cap >= 0, not NaN;
                                     EINVAL with SMILESS_FLAG_NO_PRUNE or in smiless_plan_sla_sweep */
    const int32_t *instances;     /* optional [n_funcs] host array (NULL = one instance each): NEXT-4
                                     scale-out (reading G26): function k runs
                                     instances[k] identical instances (same configuration and window);
                                     request j is dispatched to instance j mod instances[k] (round
                                     robin), each instance serves its requests in request order, and
                                     the first request of each instance finds it pre-warmed (G5).
                                     Each instance is billed for its own loaded time.
                                     1 <= instances[k] <= SMILESS_MAX_INSTANCES.  With any value > 1
                                     the throughput-mode prefix memoisation is not used (the plan runs
                                     on smiless_plan_kernel); results are exact as always.  The
                                     instance counts typically come from smiless_autoscale_rows.    */
} smiless_plan_args;

typedef struct {
    uint64_t index;           /* winning index in the suffix space; UINT64_MAX if infeasible      */
    double cost;              /* its cost sum_k U_k * E_k ($); +inf if infeasible                  */
    int64_t max_latency_us;   /* its max_j L_j; -1 if infeasible                                   */
    uint64_t n_decided;       /* candidates of this shard's range that were decided               */
    uint64_t n_full_evals;    /* candidates walked through all J arrivals                          */
    double eval_kernel_ms;    /* device time of the evaluator kernel launches (CUDA events on the
                                 launch stream)                                                    */
    double total_device_ms;   /* device time of the whole call (first upload .. last kernel)      */
    int32_t int64_path;       /* 1 if the int64 evaluator ran (int32 range check failed / forced)  */
    int32_t launches;         /* kernels this call launched                                        */
    uint64_t h2d_bytes;       /* host -> device bytes this call copied (inputs: arrivals unless on
                                 the device, windows / tables when changed, counts, caps)          */
    uint64_t d2h_bytes;       /* device -> host bytes this call copied (result block, counts,
                                 cost_out)                                                         */
    int32_t eval_path;        /* which evaluator path decided the range: SMILESS_PATH_*            */
    uint32_t n_decided_hi;    /* bits 64..95 of the decided count (smiless_plan_digits: a range of
                                 digits can hold more than 2^64 candidates, C5: 2^70); else 0     */
} smiless_plan_result;

/* smiless_plan_result.eval_path */
enum {
    SMILESS_PATH_NONE = 0,       /* nothing to search (empty range or every function pinned)      */
    SMILESS_PATH_PLAN = 1,       /* smiless_plan_kernel over the range (prune mode: compaction)    */
    SMILESS_PATH_BNB = 2,        /* branch-and-bound pre-pass + smiless_plan_kernel in list mode   */
    SMILESS_PATH_MEMO = 3,       /* throughput mode, prefix memoisation: upstream + variants kernels
                                    with the x stream through HBM                                 */
    SMILESS_PATH_MEMO_FUSED = 4  /* throughput mode, prefix memoisation in one kernel: producer warp
                                    -> shared-memory ring -> consumer warps (x stays on chip)     */
};

/* Size of the suffix candidate space prod_{k >= n_fixed} M_k * W.
 * Returns OK, ESTATE (profiles not loaded), EINVAL or ERANGE (> 2^63). */
SMILESS_API int smiless_space_size(const smiless_ctx *ctx, int32_t n_windows, int32_t n_fixed, uint64_t *out);

/* The hot path: exhaustive SLA-constrained min-cost search over [begin, end)
 * of the suffix space (this shard's chunks only when n_shards > 1).
 * config_out / window_out ([n_funcs] or NULL) receive the winner's config and
 * window index per function (the "execution strategy").
 * Returns OK, INFEASIBLE (res->index = UINT64_MAX, cost = +inf,
 * max_latency = -1, outputs set to -1), or an error. */
SMILESS_API int smiless_plan(smiless_ctx *ctx, const smiless_plan_args *a, smiless_plan_result *res,
                 int32_t *config_out, int32_t *window_out);

/* Exhaustive search over several sub-spaces in one call: every value d in [d_begin, d_end) of
 * the LAST pinned digit (a->fixed_digits[a->n_fixed - 1] is ignored), each over [begin, end) of
 * its suffix space, one after the other on the device with the running incumbent carried from
 * one digit to the next (its cost bound prunes the later digits), and one exact re-check of the
 * winner.  This is how spaces above 2^63 are planned (C5: 2^70 = 128 digits x 2^63) without a
 * host round trip per digit.  Result: the lexicographic (cost, digit, index) minimum: res->index
 * is its index in digit *digit_out's suffix space; n_decided + 2^64 n_decided_hi sums every
 * digit.  Requires 1 <= n_fixed < n_funcs, fixed_digits, 0 <= d_begin < d_end <= M * W of
 * function n_fixed - 1, and no cost_out.  Sharding (shard, n_shards) and FLAG_COST_CAP apply
 * to every digit as in smiless_plan.  digit_out (or NULL) gets -1 when nothing is feasible.
 * Returns OK, INFEASIBLE or an error. */
SMILESS_API int smiless_plan_digits(smiless_ctx *ctx, const smiless_plan_args *a, int32_t d_begin, int32_t d_end,
                                    smiless_plan_result *res, int32_t *digit_out, int32_t *config_out,
                                    int32_t *window_out);

/* The paper's adaptive pre-warming window per (function, config) row for a predicted
 * inter-arrival time it_us: Case I (T + I < IT): IT - T - I, the unloaded gap
 * that re-loads the instance exactly when the next input arrives; Case II (T + I >= IT):
 * 0, keep alive.  Host-only.  row_windows_out has sum(n_configs) entries.
 * Returns OK, ESTATE or EINVAL. */
SMILESS_API int smiless_derive_windows(const smiless_ctx *ctx, int64_t it_us, int32_t *row_windows_out);

/* NEXT-2: SMIless's own Top-1 path search (Fig. 6, Eq. (6)) -- the heuristic the
 * paper deploys -- over configurations with per-row pre-warm windows (a->row_windows_us,
 * n_windows == 1, e.g. from smiless_derive_windows; a->n_fixed must be 0).  Each function's
 * configs are ranked by the paper's per-invocation cost under adaptive pre-warming,
 * U * (T + I) in Case I and U * IT in Case II (O(N M log M)).  Root =
 * every function on its cheapest config; on an SLA miss the search walks the layers
 * F_1..F_N: in layer k functions < k keep their chosen config, functions > k run on their
 * fastest config, and F_k takes the next cheapest config until the node meets the SLA
 * (layer 1 starts at the second cheapest).  Every node is evaluated on the GPU
 * with model M (the same exact evaluator as smiless_evaluate), one batch per layer.
 * res / config_out / window_out receive the leaf (index UINT64_MAX, -1 outputs and return
 * INFEASIBLE if no node of the last layer meets the SLA); *n_nodes the evaluated nodes.
 * Returns OK, INFEASIBLE or an error. */
SMILESS_API int smiless_top1_search(smiless_ctx *ctx, const smiless_plan_args *a, int64_t it_us,
                                    smiless_plan_result *res, int32_t *config_out, int32_t *window_out,
                                    int64_t *n_nodes);

typedef struct {
    int32_t config;      /* chosen configuration (-1: none meets the target, or no invocations) */
    int64_t batch;       /* B: invocations batched per instance                                  */
    int64_t instances;   /* ceil(G / B)                                                          */
    double cost;         /* (instances * IT) * U(config): $ per time window; +inf if none         */
} smiless_autoscale_result;

/* NEXT-4: the paper's auto-scaler (Eq. (7)/(8)) for all functions at once.  For
 * function k with G_k predicted invocations in the next window of length IT and required
 * inference time target_k (I_s), choose
 *     min over (config c, B)  ceil(G_k / B) * IT * U(c)
 *     s.t.  slope_us[c] * B + intercept_us[c] <= target_k
 * where slope = lambda (alpha / x + beta) and intercept = gamma are the Eq. (1)/(2) batch model
 * of row c (x = cores or GPU share).  Per config the largest feasible B in [1, G_k] is found by
 * bisection (the constraint is monotone in B, the cost non-increasing); ties on cost go to
 * the lower config.  Doubles: slope * B then + intercept, IEEE, no FMA.  Host-only (the paper
 * reports < 0.1 ms).  Returns OK, ESTATE or EINVAL. */
SMILESS_API int smiless_autoscale(const smiless_ctx *ctx, const double *slope_us, const double *intercept_us,
                                  const int64_t *invocations, int64_t it_us, const int64_t *target_us,
                                  smiless_autoscale_result *out);

/* NEXT-4, per configuration: the Eq. (7)/(8) constraint of the auto-scaler solved for every
 * (function, configuration) row: batch_out[row] = the largest B in [1, G_k] with
 * slope_us[row] * B + intercept_us[row] <= target_us[k] (bisection; IEEE, no FMA), and
 * instances_out[row] = ceil(G_k / B); both 0 when even B = 1 misses the target or G_k <= 0.
 * The instance count of a function's fastest configuration is the smallest scale-out with
 * which it can keep up with a predicted peak of G_k invocations per window; it is what the
 * scale-out plans of smiless_plan_args.instances use (reading G26).  Host-only.
 * Returns OK, ESTATE or EINVAL. */
SMILESS_API int smiless_autoscale_rows(const smiless_ctx *ctx, const double *slope_us, const double *intercept_us,
                                       const int64_t *invocations, const int64_t *target_us, int64_t *batch_out,
                                       int64_t *instances_out);

/* NEXT-3: SMIless's handling of complex DAGs: decompose the DAG into its
 * source-to-sink paths (subgraphs with only sequential dependencies), optimise each path
 * with the Top-1 walk using the paper's O(1) closed-form latency (sum of I along the path,
 * Eq. (5)) and per-invocation cost (U (T + I) / U IT), then combine: a function on
 * several paths with different choices takes the fastest of them (the paper's rule for the
 * start/end F_s, F_e of parallel substructures), and every function on a single path is
 * moved to its cheapest config that keeps that path's closed-form latency at or below its
 * latency before combining.  Windows per row from a->row_windows_us (n_windows == 1,
 * n_fixed == 0).  The combined plan is evaluated on the GPU with model M; res /
 * config_out / window_out / *n_paths report it (INFEASIBLE if it misses the SLA under
 * model M).  At most 4096 paths. */
SMILESS_API int smiless_decompose_search(smiless_ctx *ctx, const smiless_plan_args *a, int64_t it_us,
                                         smiless_plan_result *res, int32_t *config_out, int32_t *window_out,
                                         int64_t *n_paths);

/* NEXT-3 with model M on the GPU: decompose the DAG into its source-to-sink
 * paths, plan every path exhaustively (the exact smiless_plan of the path's chain -- its own
 * functions, configurations, window grid, instances, the same arrivals and SLA -- on the GPU),
 * then combine as the paper does: a function on several paths takes the (configuration,
 * window) with the shortest inference time among the paths' choices (F_s / F_e of a parallel
 * substructure), and every function on one path only moves to its cheapest (configuration,
 * window) that keeps that path's model-M latency at or below its latency before combining
 * (paths in DFS order, functions in path order; the alternatives are evaluated on the GPU,
 * ties to the lowest digit).  The combined plan is evaluated with model M on the whole DAG
 * (res, config_out, window_out; INFEASIBLE if a path has no feasible plan or the combined plan
 * misses the SLA); *n_paths the number of paths.  a->n_fixed == 0, no row windows; at most
 * 4096 paths.  When the whole space exceeds 2^63, res->index is the plan's index with
 * function 0's digit pinned (the suffix space of functions 1..N-1); config_out / window_out
 * are always complete.  The paths are independent plans (the paper runs them in parallel,
 * P:214). */
SMILESS_API int smiless_decompose_plan(smiless_ctx *ctx, const smiless_plan_args *a, smiless_plan_result *res,
                                       int32_t *config_out, int32_t *window_out, int64_t *n_paths);

/* Multi-GPU form of smiless_decompose_plan ("the Strategy Optimizer executes the basic
 * algorithm in parallel for each subgraph"): every rank calls it with a->shard /
 * a->n_shards; each path's exhaustive plan then covers this rank's interleaved share of the
 * path's space, and after each path the library calls reduce(user, path, res) -- the caller's
 * collective, which must replace res->index / cost / max_latency_us with the ranks' global
 * lexicographic (cost, index) winner (index UINT64_MAX if no rank has a feasible one) and
 * return 0.  The library decodes that winner and every rank then combines identically.  The
 * library itself never communicates.  reduce == NULL is smiless_decompose_plan. */
typedef int (*smiless_path_reduce_fn)(void *user, int32_t path, smiless_plan_result *res);
SMILESS_API int smiless_decompose_plan_sharded(smiless_ctx *ctx, const smiless_plan_args *a,
                                               smiless_path_reduce_fn reduce, void *user, smiless_plan_result *res,
                                               int32_t *config_out, int32_t *window_out, int64_t *n_paths);

/* SLA sweep (C4: "impact of SLA settings"): ONE evaluation of the space
 * with one argmin key per SLA in slas[0..n_sla) (1 <= n_sla <= SMILESS_MAX_SLAS); pruning uses
 * their maximum; a->sla_us is ignored and a->cost_out must be NULL.  res[n_sla] and, when not
 * NULL, config_out / window_out [n_sla * n_funcs] receive each SLA's winner (index UINT64_MAX,
 * outputs -1 for an SLA nothing meets).  Returns OK or an error. */
SMILESS_API int smiless_plan_sla_sweep(smiless_ctx *ctx, const smiless_plan_args *a, const int64_t *slas,
                                       int32_t n_sla, smiless_plan_result *res, int32_t *config_out,
                                       int32_t *window_out);

/* Exact int64 evaluation (no pruning, no clamping) of n explicit candidate
 * indices of the suffix space: cost, max_j L_j and feasibility per index.
 * a->begin/end/flags(NO_PRUNE)/shard are ignored.  Returns OK or an error
 * (ERANGE if an index is outside the space). */
SMILESS_API int smiless_evaluate(smiless_ctx *ctx, const smiless_plan_args *a, const uint64_t *idx, int64_t n,
                     double *cost, int64_t *max_latency_us, uint8_t *feasible);

/* Decode a suffix-space index into per-function config and window indices
 * (pinned functions take their fixed digit).  Host-only.  Returns OK,
 * ESTATE, EINVAL or ERANGE. */
SMILESS_API int smiless_decode(const smiless_ctx *ctx, int32_t n_windows, uint64_t index, const smiless_plan_args *a,
                   int32_t *config_out, int32_t *window_out);

/* ---- introspection (build checks, SASS inspection, tests) --------------------------- */

/* Copy the NVRTC source that smiless_plan would compile for (ctx, a) into buf
 * (NUL-terminated, truncated to cap); *len receives the full size + 1.
 * Host-only.  Returns OK, EINVAL, ESTATE or ERANGE. */
SMILESS_API int smiless_kernel_source(smiless_ctx *ctx, const smiless_plan_args *a, char *buf, size_t cap,
                                      size_t *len);

/* NVRTC-compile that source for sm_100a without loading it (works without a GPU);
 * the compile/ptxas log (registers, spills) goes to log, the cubin (SASS for
 * cuobjdump) to cubin when cubin_cap is large enough; *cubin_size gets its size.
 * Returns OK, EJIT or an argument error. */
SMILESS_API int smiless_jit_compile(smiless_ctx *ctx, const smiless_plan_args *a, char *log, size_t logcap,
                                    void *cubin, size_t cubin_cap, size_t *cubin_size);

#ifdef __cplusplus
}
#endif

#endif /* SMILESS_H */
