/*
 * madpipe.h -- C ABI of the B200-native MadPipe-DP hot path (libmadpipe.so).
 *
 * The library decides, for a chain of L DNN layers, P GPUs of memory M and
 * links of bandwidth beta, the smallest candidate period tau for which the
 * memory-aware dynamic program of MadPipe (Beaumont, Eyraud-Dubois, Shilova,
 * hal-03025305, section 4.2) finds an allocation, and returns that allocation.
 * It is the "first phase" of MadPipe (Algorithm 1) with the serial
 * binary search replaced by a batched sweep over candidate periods (DESIGN.md
 * reading Q1/Q14).  "P:n" = line n of the paper text; "Qn" = DESIGN.md readings.
 *
 * Problem statement mirrored by the ABI: "finding a good load
 * balancing ... on P given processors with memory capacity M and connected via
 * the network with bandwidth beta".
 *
 * Conventions for every entry point
 *   - Return 0 (MADPIPE_OK) on success, 1 (MADPIPE_INFEASIBLE) when no candidate
 *     period admits an allocation (a valid outcome, not an error), negative on
 *     error; madpipe_last_error() then describes it.
 *   - Pointers marked [host] are host memory, [dev] are device memory on the
 *     ctx's device.  Input arrays are read-only and owned by the caller; the
 *     library keeps no pointer after return.  Output arrays are caller-allocated.
 *   - All entry points are synchronous with respect to the host (they return
 *     after their GPU work is complete) unless stated otherwise.
 *   - One ctx per host thread; a ctx is bound to one CUDA device.
 *   - Arithmetic is IEEE binary64 without FMA contraction; memory is int64
 *     bytes.  Results are bit-identical to the plain CPU oracle (oracle/).
 */
#ifndef MADPIPE_H
#define MADPIPE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MADPIPE_OK          0
#define MADPIPE_INFEASIBLE  1
#define MADPIPE_EINVAL    (-1)   /* invalid argument (see madpipe_validate)            */
#define MADPIPE_ENOMEM    (-2)   /* device or host allocation failed                    */
#define MADPIPE_ECUDA     (-3)   /* CUDA runtime error (no device, launch failure, ...) */
#define MADPIPE_ENCCL     (-4)   /* NCCL unavailable (libnccl.so.2 not loadable) or an NCCL
                                    call failed; the ctx's communicator is then unusable     */
#define MADPIPE_ESTATE    (-5)   /* call out of order (e.g. resolve of an infeasible j) */

/* A linear (or linearised) chain of L layers (section 3).
 *   uF[L], uB[L] : forward / backward duration of layer i+1 on one mini-batch,
 *                  seconds; finite, >= 0, uF+uB > 0 (reading Q9).
 *   W[L]         : weight bytes of layer i+1 (>= 0); a GPU holding it stores 3 W.
 *   a[L+1]       : activation bytes; a[0] = network input a^(0), a[l] = output of F_l
 *                  (reading Q5).  a_l is also the size of b^(l).
 * Pointers are [host] for madpipe_solve / _candidates / _dp_table / _solve_batch,
 * [dev] for madpipe_solve_dev, and either for madpipe_sweep / _resolve (the
 * library asks the CUDA runtime which; device arrays are not value-checked). */
typedef struct {
    int32_t L;
    const double  *uF;
    const double  *uB;
    const int64_t *W;
    const int64_t *a;
} madpipe_chain;

/* Range of the delay grid V (reading Q8). PAPER: 0..U(1,L)+sum C,
 * a delay beyond the range makes the transition infeasible.  SAFE:
 * 0..2(U(1,L)+sum C)+tau, saturating at the top level. */
typedef enum { MADPIPE_VRANGE_PAPER = 0, MADPIPE_VRANGE_SAFE = 1 } madpipe_vrange;

/* Discretisation (the paper uses 11 memory levels and 51 delay levels). */
typedef struct {
    int32_t n_mem;      /* levels of the special GPU's memory m_P in [0,M], 2..64       */
    int32_t n_delay;    /* levels of the delay V, 2..65535                               */
    int32_t n_periods;  /* candidate periods, uniform on [lb, ub] (P:205 l.1-2, Q14), >= 1 */
    int32_t v_range;    /* madpipe_vrange                                                 */
    int32_t early_exit; /* 0: evaluate every candidate; 1: ascending, stop at the first
                           feasible one (exact); 2: coarse-to-fine (every ~sqrt(n_periods)-th
                           candidate, then the gap below the first feasible one; equal to
                           the full sweep when feasibility is monotone in the period, P:199;
                           madpipe_solve / _solve_dev only -- elsewhere 2 acts as 1)        */
} madpipe_disc;

/* Result of a solve (the decisions along the optimal path give the
 * partitioning and the assignment).  Stages are in chain order; stage_proc is
 * in [0, P-2] for the normal GPUs (numbered in chain order) and P-1 for the
 * special GPU.  The three stage arrays are caller-allocated with
 * capacity L; the library writes n_stages entries. */
typedef struct {
    double   period;        /* tau_{j*}: the candidate period found (Alg. 1 step 5, Q16)   */
    double   load_period;   /* load of the most loaded GPU or link, <= period       */
    double   special_load;  /* DP root value A[L][P-1][0][0]: the special GPU's load         */
    int32_t  cand_index;    /* j* (or -1 if infeasible)                                      */
    int32_t  n_stages;
    int32_t *stage_first;   /* [host] capacity L, 1-based first layer                        */
    int32_t *stage_last;    /* [host] capacity L, 1-based last layer                         */
    int32_t *stage_proc;    /* [host] capacity L                                              */
    int64_t  cell_updates;  /* relaxations evaluated by the sweep             */
} madpipe_alloc;

typedef struct madpipe_ctx madpipe_ctx;

/* ---- context --------------------------------------------------------------
 * One process per GPU.  A ctx is bound to CUDA
 * device `device` and is rank `rank` of `world` ranks.  With world > 1 the ctx
 * owns an NCCL communicator built from `nccl_id` (128 bytes from
 * madpipe_get_unique_id on one rank, distributed by the caller -- process
 * bootstrap only), over which madpipe_solve / _solve_dev / _solve_batch run
 * the path's single exchange step a7 (the MIN all-reduce of the candidate
 * indices) themselves: an N-GPU solve is one call per rank, every rank passes
 * identical inputs and receives the identical result.  With world = 1,
 * `nccl_id` may be NULL (no communicator) or a valid id (a communicator of one
 * rank: the same collective code path, e.g. for tests on one GPU).
 * `cuda_stream` is a cudaStream_t to issue work on (e.g.
 * torch.cuda.current_stream().cuda_stream), or NULL for a stream owned by the
 * ctx.  `mem_budget` bounds the device bytes used for DP tables (0 = 60% of the
 * free memory at creation).  Errors: MADPIPE_EINVAL (rank/world/device),
 * MADPIPE_ECUDA (no usable device), MADPIPE_ENCCL (NCCL missing or
 * ncclCommInitRank failed).  NCCL is loaded at run time (dlopen of
 * libnccl.so.2, or MADPIPE_NCCL_LIB). */
int  madpipe_get_unique_id(uint8_t id[128]);
int  madpipe_ctx_create(madpipe_ctx **out, int device, int32_t rank, int32_t world,
                        const uint8_t *nccl_id, void *cuda_stream, int64_t mem_budget);
void madpipe_ctx_destroy(madpipe_ctx *ctx);
const char *madpipe_last_error(const madpipe_ctx *ctx);   /* ctx may be NULL */
/* rank, world and the loaded NCCL version (0 = no communicator); any may be NULL. */
int  madpipe_ctx_info(const madpipe_ctx *ctx, int32_t *rank, int32_t *world, int32_t *nccl_version);

/* ---- host-only helpers (no GPU needed) ------------------------------------ */
/* Check every argument rule of this header; MADPIPE_OK or MADPIPE_EINVAL.
 * Rules: L >= 1; P >= 1; M > 0; beta > 0 and not NaN (beta = +inf allowed:
 * C = 0); uF, uB finite, >= 0, uF+uB > 0; W >= 0; a >= 0; 2 <= n_mem <= 64;
 * 2 <= n_delay <= 65535; n_periods >= 1; v_range in {0,1}; int64 overflow
 * guards 3*sum W + (g_max)*sum a and (M-1) + (n_mem-1)*(3 sum W + g_max sum a). */
int madpipe_validate(const madpipe_chain *chain, int32_t P, int64_t M, double beta,
                     const madpipe_disc *disc);
/* Candidates owned by `rank` of `world` (interleaved: j = rank, rank+world, ...;
 * DESIGN.md 7).  Writes up to n_periods indices into out[] and their count. */
int madpipe_shard(int32_t n_periods, int32_t rank, int32_t world, int32_t *out, int32_t *count);
/* Exact number of cell-updates of candidate period tau:
 * sum_l (l - kmin(l) + 1) (P-1) n_delay n_mem, where kmin(l) is the smallest k
 * with U(k,l) <= tau.  [host] chain. */
int64_t madpipe_cell_updates(const madpipe_chain *chain, int32_t P, const madpipe_disc *disc,
                             double tau);

/* ---- the hot path -----------------------------------------------------------
 * Full solve: profile prep (a1), candidate grid (a2), the batched wavefront DP
 * over this rank's candidates (a3-a5; rank r of W owns j = r, r+W, ..., as
 * madpipe_shard), root test and local minimum (a6), the MIN all-reduce of the
 * ranks' smallest feasible index over the ctx's communicator (a7; skipped
 * without one), winner re-solve and device traceback on every rank (a8),
 * result (a9).  With disc->early_exit = 2 each of the two rounds (coarse, then
 * the gap) is split over the ranks and ends in one all-reduce.
 * out->cell_updates counts this rank's relaxations.  [host] chain and output. */
int madpipe_solve(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                  double beta, const madpipe_disc *disc, madpipe_alloc *out);
/* Same, with the chain arrays already resident in device memory ([dev]). */
int madpipe_solve_dev(madpipe_ctx *ctx, const madpipe_chain *chain_dev, int32_t P, int64_t M,
                      double beta, const madpipe_disc *disc, madpipe_alloc *out);

/* The two halves of a multi-GPU solve, for a rank `rank` of `world` given
 * explicitly (independent of the ctx's own rank/world; no collective): what
 * madpipe_solve does around its all-reduce, exposed for tests and for callers
 * with their own transport.  madpipe_sweep evaluates that rank's shard of
 * candidates and writes the smallest feasible candidate index it owns
 * (INT32_MAX if none) to *j_local [dev, int32]; the min over ranks, passed to
 * madpipe_resolve [dev, int32], is re-solved and traced back; every rank gets
 * the same result.  cell_updates_out [host] receives the shard's relaxation
 * count.  With disc->early_exit the rank stops at its first feasible candidate. */
int madpipe_sweep(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                  double beta, const madpipe_disc *disc, int32_t rank, int32_t world,
                  int32_t *j_local, int64_t *cell_updates_out);
int madpipe_resolve(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                    double beta, const madpipe_disc *disc, const int32_t *j_star,
                    madpipe_alloc *out);

/* Batch of n independent chains (BASELINE config 5, the paper's evaluation
 * grid P:235) with per-chain P[i], M[i], beta[i] and a shared discretisation;
 * out[i] as for madpipe_solve (cand_index -1 for an infeasible chain).  All
 * (chain, candidate) pairs form one work list.  At world > 1 the list is split
 * over the ranks by LPT on each pair's cell-update count (madpipe_batch_plan),
 * the ranks MIN-all-reduce an int32[n] of per-chain smallest feasible indices
 * (a7), each winner is re-solved by one owner (madpipe_resolve_plan) and the
 * fixed-size results are all-gathered, so every rank returns all n results.
 * out[i].cell_updates counts this rank's relaxations of chain i.  Returns
 * MADPIPE_OK if the call succeeded.  [host]. */
int madpipe_solve_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains,
                        const int32_t *P, const int64_t *M, const double *beta,
                        const madpipe_disc *disc, madpipe_alloc *out);
/* Building blocks of the batch at rank `rank` of `world` (independent of the
 * ctx's own rank/world; no collective): madpipe_sweep_batch evaluates the jobs
 * the plan gives this rank and writes j_local[n] [host] (INT32_MAX where this
 * rank found none) and cell_updates_out[n] [host, may be NULL];
 * madpipe_resolve_batch re-solves the winners j_star[n] [host] (INT32_MAX =
 * infeasible) this rank owns and writes only those out[i].  The element-wise
 * MIN of the ranks' j_local is what madpipe_solve_batch all-reduces. */
int madpipe_sweep_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains, const int32_t *P,
                        const int64_t *M, const double *beta, const madpipe_disc *disc, int32_t rank,
                        int32_t world, int32_t *j_local, int64_t *cell_updates_out);
int madpipe_resolve_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains, const int32_t *P,
                          const int64_t *M, const double *beta, const madpipe_disc *disc,
                          const int32_t *j_star, int32_t rank, int32_t world, madpipe_alloc *out);
/* Host-only (no GPU): the batch work plan over `world` ranks.  owner[n*n_periods]
 * (may be NULL): owner[i*n_periods + j] = rank evaluating candidate j of chain i;
 * load[world] (may be NULL): each rank's summed cost; cost[n*n_periods] (may be
 * NULL): the cost of each pair = its cell-updates + (L+1) n_delay P.
 * LPT: pairs by decreasing cost (ties: lower index), each to the least-loaded rank
 * (ties: lower rank); deterministic, so every rank computes the same plan.
 * madpipe_resolve_plan: owner[n] of each winner's re-solve (LPT on the winners'
 * costs; -1 where j_star[i] = INT32_MAX). [host] chains (uF, uB, a read). */
int madpipe_batch_plan(int32_t n, const madpipe_chain *chains, const int32_t *P, const double *beta,
                       const madpipe_disc *disc, int32_t world, int32_t *owner, int64_t *load,
                       int64_t *cost);
int madpipe_resolve_plan(int32_t n, const madpipe_chain *chains, const int32_t *P, const double *beta,
                         const madpipe_disc *disc, const int32_t *j_star, int32_t world, int32_t *owner);

/* ---- parity / debug exports (small configs) ------------------------------- */
/* Every candidate's period tau_out[n_periods] and root value root_out[n_periods]
 * (A_j[L][P-1][0][0]; +inf if infeasible). [host]. */
int madpipe_candidates(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                       double beta, const madpipe_disc *disc, double *tau_out, double *root_out);
/* Full DP table of candidate j, A_out[(L+1)*P*n_delay*n_mem] in [l][p][v][m]
 * order, and the decision arg_out (same shape, may be NULL): 2k+o with o = 1
 * for the special GPU, -1 where the cell is infeasible (tie-break Q11). [host]. */
int madpipe_dp_table(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                     double beta, const madpipe_disc *disc, int32_t j, double *A_out,
                     int32_t *arg_out);

/* Timing of the last solve/sweep on the ctx's stream (CUDA events): total
 * milliseconds of the sweep kernels, of the dominant step kernel alone, and
 * the number of kernel launches issued. */
int madpipe_last_timing(const madpipe_ctx *ctx, double *sweep_ms, double *step_kernel_ms,
                        int64_t *launches);
/* per_launch = 1: bracket every step-kernel launch with CUDA events so that
 * madpipe_last_timing reports the step kernel's own time (bench roofline);
 * 0 (default): only the sweep is timed. */
int madpipe_set_timing(madpipe_ctx *ctx, int per_launch);
/* Bytes the last call copied host->device and device->host (inputs, job
 * descriptors, results); for the bench's end-to-end record. */
int madpipe_last_io(const madpipe_ctx *ctx, int64_t *h2d_bytes, int64_t *d2h_bytes);
/* Relaxation counts of the last sweep: cell_updates as in
 * madpipe_alloc (every (k, l, v, p, m) of the tau-windows); effective_updates,
 * the relaxations whose transition is live (not skipped by a delay overflow, a
 * communication longer than the period, or neither N nor S fitting); and
 * useful_updates, the live ones whose source row holds a finite value -- the
 * ones the default step kernel reads (0 for the other step kernels). */
int madpipe_last_counts(const madpipe_ctx *ctx, int64_t *cell_updates, int64_t *effective_updates,
                        int64_t *useful_updates);
/* Algorithmic bytes of the step kernel in the last sweep, the
 * numerator of the bench's roofline: load_bytes = every source-row segment the
 * step kernel brings on chip ((np+1) processor rows of the padded n_mem levels,
 * fp64, per processor tile; the two-layer kernel loads a row shared by both of
 * its layers once), store_bytes = every output row p >= 1 it writes.  segments =
 * the number of merged source segments of the two-layer kernel (0 otherwise).
 * Host-computed from the device counters; no GPU access. */
int madpipe_last_step_bytes(const madpipe_ctx *ctx, int64_t *load_bytes, int64_t *store_bytes,
                            int64_t *segments);
/* Step kernel that ran the largest batch of the last sweep:
 * 0 = plain-load step_kernel, 2 = persistent
 * single-layer step_persist_kernel, 3 = persistent two-layer pair_step_kernel.
 * Chosen per batch from the row-segment size unless MADPIPE_KERNEL forces one.
 * Host only. */
int madpipe_last_kernel(const madpipe_ctx *ctx, int32_t *kernel);

/* ---- NEXT row f2: the 1F1B* pattern of a contiguous allocation (host only) --
 * For stages s_1..s_N (one per GPU, tiling layers 1..L in order; e.g. a
 * madpipe_alloc whose special GPU holds at most one stage) and a period T:
 * the 2N-1 item chain of stages and communications, its 1F1B* groups
 * and the periodic pattern: for every item its forward and
 * backward start time in [0, T), index shift h (in period k the operation
 * processes batch k-h) and duration.  Item i of group g keeps g activations
 * alive.  ops[] is caller-allocated with capacity 2N-1.
 * Returns MADPIPE_INFEASIBLE if an item's load exceeds T, MADPIPE_EINVAL for
 * stages that do not tile the chain. */
typedef struct {
    int32_t kind;       /* 0 = stage (GPU), 1 = communication (link)                 */
    int32_t stage;      /* stage index (for a communication: the stage it feeds)      */
    int32_t group;      /* 1F1B* group, 1 = the group holding the last stage          */
    int32_t f_shift;    /* index shift of the forward operation                       */
    int32_t b_shift;    /* index shift of the backward operation                      */
    int32_t pad_;
    double  f_start, f_len, b_start, b_len;   /* seconds; starts in [0, T)             */
} madpipe_op;
int madpipe_schedule(const madpipe_chain *chain, double beta, double period, int32_t n_stages,
                     const int32_t *stage_first, const int32_t *stage_last, madpipe_op *ops,
                     int32_t *n_ops);

/* ---- NEXT row f1: the paper-literal MadPipe-DP and Algorithm 1 --------------
 * The serial baseline the candidate sweep replaces: K = 10 calls
 * of the optimisation-form DP T(l, p, t_P, m_P, V) with
 * t_P discretised into n_tp levels on [0, U(1,L)] (101), m_P into n_mem
 * and V into n_delay levels (PAPER range), driven by the modified binary search
 * of Algorithm 1 (reading Q15).  out->period = min_i max(T_i, That_i)
 * (P:199), out->cand_index = that i, the stages come from a device traceback of
 * DP(That_i) (tie-break Q11); T_hist / That_hist [host, K] (may be NULL) get
 * every iteration.  cell_updates is 0 (not a sweep).  [host] chain. */
int madpipe_solve_paper(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M, double beta,
                        int32_t n_mem, int32_t n_delay, int32_t n_tp, int32_t K, madpipe_alloc *out,
                        double *T_hist, double *That_hist);
/* The literal DP table at target That: A_out[(L+1)*P*n_tp*n_delay*n_mem] in
 * [l][p][t][v][m] order and its decisions (may be NULL), for parity tests. */
int madpipe_literal_table(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M, double beta,
                          int32_t n_mem, int32_t n_delay, int32_t n_tp, double That, double *A_out,
                          int32_t *arg_out);

#ifdef __cplusplus
}
#endif
#endif /* MADPIPE_H */
