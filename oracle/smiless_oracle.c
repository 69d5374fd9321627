/*
 * oracle/smiless_oracle.c -- the plain CPU oracle for the SMIless
 * co-optimisation hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or constant with the CUDA path
 * (paper_conf_sc_luxl0y024_b200/), and it never reads anything the CUDA path
 * produced.
 *
 * What it computes (citations are PAPER.md line numbers, "P:n"):
 *
 *   OPT = argmin over all candidates (chi, phi) of  sum_k C_k(*_k, /\_k)
 *         subject to  L(chi, phi) <= SLA                  P:160 Eq. (4)
 *   C_k = E_k(*_k, /\_k) * U(*_k)                         P:156 Eq. (3)
 *   E_k = init + inference + keep-alive time
 *
 * where E_k and L come from simulating every predicted invocation through the
 * DAG with model M, which extends the
 * paper's Case I / II / III rules from periodic arrivals to an
 * arbitrary predicted arrival sequence.  Readings of silent/garbled passages
 * (G1-G20) are listed in DESIGN.md.
 *
 * Deliberately naive: int64 ABSOLUTE times, a literal case split per
 * invocation, per-step billing, the full D[k][j] matrix, no pruning, no early
 * exit, no algebraic reformulation, brute force over the index range.
 * Floating point: cost = ((U0*b0 + U1*b1) + U2*b2) + ...  left to right,
 * each mul and add correctly rounded; compiled with -ffp-contract=off so no
 * FMA contraction happens.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

typedef struct {
    int32_t n_funcs;
    const int32_t *pred_ptr;     /* [N+1] topologically ordered predecessor CSR */
    const int32_t *pred_idx;     /* [E]                                          */
    const int32_t *n_configs;    /* [N]   M_k                                    */
    const int32_t *exec_us;      /* [sum M] I[k][c]                     */
    const int32_t *init_us;      /* [sum M] T[k][c]  (P:175, P:120 mu+3sigma)    */
    const double *price_per_us;  /* [sum M] U[k][c]              */
    const int64_t *arrivals_us;  /* [J]   r_0 <= ... <= r_{J-1}       */
    int64_t n_arrivals;          /* J >= 1                                       */
    int64_t sla_us;
    const int32_t *windows_us;   /* [W]   policy set S; 0 = keep-alive    */
    int32_t n_windows;
    int32_t n_fixed;             /* digits of functions 0..n_fixed-1 are pinned   */
    const int32_t *fixed_digits; /* [n_fixed] digit = config * W + window         */
    const int32_t *row_windows;  /* optional [sum M]: the window of (k, c) itself  */
                                 /* (NEXT-1 derived windows; then W must be 1)    */
    const int32_t *instances;    /* optional [N]: n_k >= 1 instances of function k */
                                 /* (NEXT-4 scale-out, reading G26); NULL = all 1  */
} oracle_problem;

/* Row offset of function k in the function-major profile arrays. */
static int64_t row0(const oracle_problem *P, int k) {
    int64_t o = 0;
    for (int i = 0; i < k; ++i) o += P->n_configs[i];
    return o;
}

/* Size of the (suffix) candidate space: prod_{k >= n_fixed} M_k * W.
   Returns 0 above 2^63 (every index must fit an int64). */
uint64_t oracle_space_size(const oracle_problem *P) {
    unsigned __int128 s = 1;
    for (int k = P->n_fixed; k < P->n_funcs; ++k) {
        s *= (unsigned __int128)((uint64_t)P->n_configs[k] * (uint64_t)P->n_windows);
        if (s > ((unsigned __int128)1 << 63)) return 0;
    }
    return (uint64_t)s;
}

/* Mixed-radix decode.  index = sum_k d_k * S_k over the suffix functions,
   function n_fixed most significant, d_k = c_k * W + w_k (config major). */
void oracle_decode(const oracle_problem *P, uint64_t index, int32_t *config, int32_t *window) {
    const int N = P->n_funcs, W = P->n_windows;
    for (int k = N - 1; k >= P->n_fixed; --k) {
        uint64_t radix = (uint64_t)P->n_configs[k] * (uint64_t)W;
        uint64_t d = index % radix;
        index /= radix;
        config[k] = (int32_t)(d / (uint64_t)W);
        window[k] = (int32_t)(d % (uint64_t)W);
    }
    for (int k = 0; k < P->n_fixed; ++k) {
        config[k] = P->fixed_digits[k] / W;
        window[k] = P->fixed_digits[k] % W;
    }
}

/* A function is a sink when no function lists it as a predecessor. */
static void find_sinks(const oracle_problem *P, uint8_t *is_sink) {
    for (int k = 0; k < P->n_funcs; ++k) is_sink[k] = 1;
    for (int e = 0; e < P->pred_ptr[P->n_funcs]; ++e) is_sink[P->pred_idx[e]] = 0;
}

/*
 * Model M for one candidate.  D is caller scratch of N*J int64.
 * Outputs: billed[k] (int64 us, the E_k of Eq. (3)), latency[j] = L_j.
 *
 *   x   = r_j                          for a source function
 *       = max_{p in pred(k)} D[p][j]   otherwise   (AND-join; "max over
 *                                        parallel branches")
 *   Scale-out (NEXT-4, "launching multiple instances of the same function";
 *   reading G26): function k runs n_k identical instances (same configuration and
 *   window); request j is served by instance j mod n_k (round-robin dispatch), each
 *   instance in request order.  n_k = 1 is the single instance of P:169-200.
 *
 *   j <  n_k:  start = x, bill = T   (first invocation on its instance pre-warmed, G5)
 *   j >= n_k, f = D[k][j-n_k] (previous completion on this instance), g = x - f:
 *     g <= 0       : start = f,   bill = 0      busy -> FIFO wait, stays warm
 *                                               (Case III, Fig. 5(c); G6)
 *     window == 0  : start = x,   bill = g      keep-alive, idle time billed
 *                                               (Case II; G10)
 *     else s = f + window  (unloaded for `window` after completion, then the
 *                           pre-warm init of length T starts; Case I, P:177;
 *                           readings G1, G2)
 *       x <  s     : start = x+T, bill = T      pre-warm not begun: cold start
 *                                               on arrival (G3)
 *       x <  s+T   : start = s+T, bill = T      init partly covered: wait (G4)
 *       otherwise  : start = x,   bill = x - s  init T + loaded idle x-s-T (G7)
 *   D[k][j] = start + I;  billed[k] += bill + I
 *   L_j = max_{sink} D[sink][j] - r_j                                (G8)
 */
static void simulate_into(const oracle_problem *P, const int32_t *config, const int32_t *window,
                          const uint8_t *is_sink, int64_t *D, int64_t *billed, int64_t *latency) {
    const int N = P->n_funcs;
    const int64_t J = P->n_arrivals;
    const int64_t *r = P->arrivals_us;
    int64_t I[64], T[64], w[64], n_inst[64];
    for (int k = 0; k < N; ++k) {
        n_inst[k] = P->instances ? P->instances[k] : 1;
        int64_t row = row0(P, k) + config[k];
        I[k] = P->exec_us[row];
        T[k] = P->init_us[row];
        w[k] = P->row_windows ? P->row_windows[row] : P->windows_us[window[k]];
        billed[k] = 0;
    }
    for (int64_t j = 0; j < J; ++j) {
        for (int k = 0; k < N; ++k) {
            int64_t x;
            if (P->pred_ptr[k] == P->pred_ptr[k + 1]) {
                x = r[j];
            } else {
                x = D[(int64_t)P->pred_idx[P->pred_ptr[k]] * J + j];
                for (int e = P->pred_ptr[k] + 1; e < P->pred_ptr[k + 1]; ++e) {
                    int64_t v = D[(int64_t)P->pred_idx[e] * J + j];
                    if (v > x) x = v;
                }
            }
            int64_t start, bill;
            if (j < n_inst[k]) {
                start = x;
                bill = T[k];
            } else {
                int64_t f = D[(int64_t)k * J + (j - n_inst[k])];
                int64_t g = x - f;
                if (g <= 0) {
                    start = f;
                    bill = 0;
                } else if (w[k] == 0) {
                    start = x;
                    bill = g;
                } else {
                    int64_t s = f + w[k];
                    if (x < s) {
                        start = x + T[k];
                        bill = T[k];
                    } else if (x < s + T[k]) {
                        start = s + T[k];
                        bill = T[k];
                    } else {
                        start = x;
                        bill = x - s;
                    }
                }
            }
            D[(int64_t)k * J + j] = start + I[k];
            billed[k] += bill + I[k];
        }
        int64_t lat = INT64_MIN;
        for (int k = 0; k < N; ++k)
            if (is_sink[k]) {
                int64_t v = D[(int64_t)k * J + j] - r[j];
                if (v > lat) lat = v;
            }
        latency[j] = lat;
    }
}

/* cost = sum_k U[k][c_k] * billed[k], k = 0..N-1 left to right (Eq. 3, 4). */
static double cost_of(const oracle_problem *P, const int32_t *config, const int64_t *billed) {
    double cost = 0.0;
    for (int k = 0; k < P->n_funcs; ++k) {
        double u = P->price_per_us[row0(P, k) + config[k]];
        double term = u * (double)billed[k];
        cost = cost + term;
    }
    return cost;
}

/* Public: simulate one explicit candidate.  Returns 0, or -1 on bad args. */
/* instances, when given, must be >= 1 */
static int bad_problem(const oracle_problem *P) {
    if (P->n_funcs < 1 || P->n_funcs > 64 || P->n_arrivals < 1) return 1;
    if (P->instances)
        for (int k = 0; k < P->n_funcs; ++k)
            if (P->instances[k] < 1) return 1;
    return 0;
}

int oracle_simulate(const oracle_problem *P, const int32_t *config, const int32_t *window,
                    int64_t *billed, int64_t *latency) {
    if (bad_problem(P)) return -1;
    uint8_t is_sink[64];
    find_sinks(P, is_sink);
    int64_t *D = (int64_t *)malloc(sizeof(int64_t) * (size_t)P->n_funcs * (size_t)P->n_arrivals);
    if (!D) return -1;
    simulate_into(P, config, window, is_sink, D, billed, latency);
    free(D);
    return 0;
}

typedef struct {
    const oracle_problem *P;
    const uint8_t *is_sink;
    int64_t *D, *billed, *latency;
    int32_t config[64], window[64];
} worker_scratch;

static int scratch_init(worker_scratch *s, const oracle_problem *P, const uint8_t *is_sink) {
    s->P = P;
    s->is_sink = is_sink;
    s->D = (int64_t *)malloc(sizeof(int64_t) * (size_t)P->n_funcs * (size_t)P->n_arrivals);
    s->billed = (int64_t *)malloc(sizeof(int64_t) * (size_t)P->n_funcs);
    s->latency = (int64_t *)malloc(sizeof(int64_t) * (size_t)P->n_arrivals);
    return (s->D && s->billed && s->latency) ? 0 : -1;
}

static void scratch_free(worker_scratch *s) {
    free(s->D);
    free(s->billed);
    free(s->latency);
}

/* Evaluate candidate `index`: cost, max_j L_j, feasible = (max L <= SLA). */
static void eval_one(worker_scratch *s, uint64_t index, double *cost, int64_t *max_lat, uint8_t *feasible) {
    const oracle_problem *P = s->P;
    oracle_decode(P, index, s->config, s->window);
    simulate_into(P, s->config, s->window, s->is_sink, s->D, s->billed, s->latency);
    int64_t m = INT64_MIN;
    for (int64_t j = 0; j < P->n_arrivals; ++j)
        if (s->latency[j] > m) m = s->latency[j];
    *max_lat = m;
    *feasible = (uint8_t)(m <= P->sla_us);
    *cost = cost_of(P, s->config, s->billed);
}

int oracle_evaluate(const oracle_problem *P, const uint64_t *idx, int64_t n,
                    double *cost, int64_t *max_lat, uint8_t *feasible) {
    if (bad_problem(P)) return -1;
    uint8_t is_sink[64];
    find_sinks(P, is_sink);
    worker_scratch s;
    if (scratch_init(&s, P, is_sink)) { scratch_free(&s); return -1; }
    for (int64_t i = 0; i < n; ++i) eval_one(&s, idx[i], &cost[i], &max_lat[i], &feasible[i]);
    scratch_free(&s);
    return 0;
}

typedef struct {
    worker_scratch s;
    uint64_t begin, end;
    int found;
    uint64_t best_idx;
    double best_cost;
    int64_t best_lat;
    int failed;
} plan_job;

static void *plan_worker(void *arg) {
    plan_job *job = (plan_job *)arg;
    job->found = 0;
    for (uint64_t i = job->begin; i < job->end; ++i) {
        double c;
        int64_t m;
        uint8_t ok;
        eval_one(&job->s, i, &c, &m, &ok);
        /* strict < in increasing index order keeps the lowest index on ties (G12) */
        if (ok && (!job->found || c < job->best_cost)) {
            job->found = 1;
            job->best_cost = c;
            job->best_idx = i;
            job->best_lat = m;
        }
    }
    return NULL;
}

/*
 * Brute force over [begin, end) of the (suffix) space (end == 0 -> all).
 * Threads take contiguous chunks; their results are combined in chunk order
 * with strict <, which is the same as one sequential scan.
 * Returns 1 (found), 0 (nothing feasible), -1 (bad args).
 */
int oracle_plan(const oracle_problem *P, uint64_t begin, uint64_t end, int n_threads,
                uint64_t *best_idx, double *best_cost, int64_t *best_lat) {
    if (bad_problem(P)) return -1;
    uint64_t space = oracle_space_size(P);
    if (space == 0) return -1;
    if (end == 0 || end > space) end = space;
    if (begin >= end) return 0;
    if (n_threads < 1) n_threads = 1;
    if ((uint64_t)n_threads > end - begin) n_threads = (int)(end - begin);
    uint8_t is_sink[64];
    find_sinks(P, is_sink);
    plan_job *jobs = (plan_job *)calloc((size_t)n_threads, sizeof(plan_job));
    pthread_t *th = (pthread_t *)calloc((size_t)n_threads, sizeof(pthread_t));
    uint64_t total = end - begin;
    int rc = 0;
    for (int t = 0; t < n_threads; ++t) {
        jobs[t].begin = begin + total * (uint64_t)t / (uint64_t)n_threads;
        jobs[t].end = begin + total * (uint64_t)(t + 1) / (uint64_t)n_threads;
        if (scratch_init(&jobs[t].s, P, is_sink)) rc = -1;
    }
    if (rc == 0) {
        for (int t = 0; t < n_threads; ++t) pthread_create(&th[t], NULL, plan_worker, &jobs[t]);
        for (int t = 0; t < n_threads; ++t) pthread_join(th[t], NULL);
        int found = 0;
        for (int t = 0; t < n_threads; ++t) {
            if (jobs[t].found && (!found || jobs[t].best_cost < *best_cost)) {
                found = 1;
                *best_cost = jobs[t].best_cost;
                *best_idx = jobs[t].best_idx;
                *best_lat = jobs[t].best_lat;
            }
        }
        rc = found;
    }
    for (int t = 0; t < n_threads; ++t) scratch_free(&jobs[t].s);
    free(jobs);
    free(th);
    return rc;
}
