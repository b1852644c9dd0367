/*
 * madpipe_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU oracle for the MadPipe memory-aware DP
 * (Beaumont, Eyraud-Dubois, Shilova, "MadPipe: Memory Aware Dynamic Programming
 * Algorithm for Pipelined Model Parallelism", hal-03025305).  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this file.  It shares no code, header, table or constant with the
 * CUDA product library (paper_conf_ipps_beaumontes22_b200/csrc); neither
 * includes the other.
 *
 * Citations: "P:n" = line n of the paper text; "Qn"/"On" = the
 * readings / normative steps listed in DESIGN.md section 3 (taken from
 * SURVEY.md section 8(c)).
 *
 * Arithmetic: IEEE-754 binary64, round to nearest even, NO FMA contraction
 * (compile with -ffp-contract=off, never -ffast-math).  Memory is int64 bytes.
 *
 * Layer indices are 1-based as in the paper (layers 1..L).  Host arrays:
 *   uF[L], uB[L], W[L]  : entry i-1 holds layer i
 *   a[L+1]              : a[0] = network input a^(0), a[l] = output of F_l
 *
 * The DP is evaluated in its decision form (reading Q1): for a target period
 * tau (= T-hat), A[l][p][v][m] is the smallest special-processor load of an
 * allocation of layers 1..l to p normal processors + the special one, with
 * every normal stage load, every boundary communication and the special load
 * all <= tau, given delay level v (V = v*dV) after F_l and special memory
 * level m (m*M/(n_m-1) already used).  +inf = infeasible.
 *
 * Parity status: pinned (brute force O11, special cases O13, invariants via
 * the 1F1B* simulator O10; see tests/test_oracle_*.py).  Parity with numbers
 * printed in the paper: UNPINNED -- the paper prints no worked example and no
 * numeric table (all figures stripped, P:209/P:227/P:239).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define OR_OK 0
#define OR_INFEASIBLE 1
#define OR_EINVAL (-1)
#define OR_ENOMEM (-2)

#define VR_PAPER 0
#define VR_SAFE 1

#define VN_OVERFLOW (-1)

typedef struct {
    int L, P, n_m, n_v, v_range;
    int64_t M;
    double beta;
    const int64_t *W, *a;
    double *Up;      /* [L+1] O1: Up[i] = Up[i-1] + (uF_i + uB_i)  */
    int64_t *Wp;     /* [L+1] Wp[i] = Wp[i-1] + W_i  */
    int64_t *Ap;     /* [L+1] Ap[i] = Ap[i-1] + a_{i-1}  */
    double *C;       /* [L+1] C[i] = 2 a_i / beta, i=1..L-1; C[0]=0 (Q3) */
    double SC;       /* sum_{i=1}^{L-1} C[i] (reading Q4)  */
} chain_t;

/* ---------------------------------------------------------------- O1 */
static int chain_init(chain_t *c, int L, const double *uF, const double *uB,
                      const int64_t *W, const int64_t *a, int P, int64_t M,
                      double beta, int n_m, int n_v, int v_range)
{
    memset(c, 0, sizeof(*c));
    if (L < 1 || P < 1 || M <= 0 || !(beta > 0.0) || n_m < 2 || n_v < 2)
        return OR_EINVAL;
    for (int i = 0; i < L; i++) {
        if (!isfinite(uF[i]) || !isfinite(uB[i]) || uF[i] < 0.0 || uB[i] < 0.0 ||
            !(uF[i] + uB[i] > 0.0) || W[i] < 0)
            return OR_EINVAL;
    }
    for (int i = 0; i <= L; i++)
        if (a[i] < 0) return OR_EINVAL;
    c->L = L; c->P = P; c->M = M; c->beta = beta;
    c->n_m = n_m; c->n_v = n_v; c->v_range = v_range;
    c->W = W; c->a = a;
    c->Up = (double *)calloc((size_t)L + 1, sizeof(double));
    c->Wp = (int64_t *)calloc((size_t)L + 1, sizeof(int64_t));
    c->Ap = (int64_t *)calloc((size_t)L + 1, sizeof(int64_t));
    c->C = (double *)calloc((size_t)L + 1, sizeof(double));
    if (!c->Up || !c->Wp || !c->Ap || !c->C) return OR_ENOMEM;
    c->Up[0] = 0.0; c->Wp[0] = 0; c->Ap[0] = 0;
    for (int i = 1; i <= L; i++) {
        c->Up[i] = c->Up[i - 1] + (uF[i - 1] + uB[i - 1]);
        c->Wp[i] = c->Wp[i - 1] + W[i - 1];
        c->Ap[i] = c->Ap[i - 1] + a[i - 1];
    }
    c->C[0] = 0.0;
    c->SC = 0.0;
    for (int i = 1; i <= L - 1; i++) {
        c->C[i] = (2.0 * (double)a[i]) / beta;
        c->SC = c->SC + c->C[i];
    }
    c->C[L] = 0.0; /* never used: no communication after the last layer */
    return OR_OK;
}

static void chain_free(chain_t *c)
{
    free(c->Up); free(c->Wp); free(c->Ap); free(c->C);
    memset(c, 0, sizeof(*c));
}

/* U(k,l) = sum_{i=k..l} (uF_i + uB_i), as a prefix difference (Q13). */
static double U(const chain_t *c, int k, int l) { return c->Up[l] - c->Up[k - 1]; }

/* ---------------------------------------------------------------- O2
 * M(k,l,g) = sum_{i=k..l}(3 W_i + g a_{i-1}) + 2(a_{k-1} + a_l), dropping the
 * buffer term at k=1 and at l=L (section 4.2.1). */
static int64_t Mem(const chain_t *c, int k, int l, int64_t g)
{
    int64_t m = 3 * (c->Wp[l] - c->Wp[k - 1]) + g * (c->Ap[l] - c->Ap[k - 1]);
    if (k > 1) m += 2 * c->a[k - 1];
    if (l < c->L) m += 2 * c->a[l];
    return m;
}

/* ---------------------------------------------------------------- O4
 * x (+) y: x + y if ceil(x/T) == ceil((x+y)/T), else T*ceil(x/T) + y. */
double oracle_oplus(double x, double y, double tau)
{
    double cx = ceil(x / tau);
    double s = x + y;
    if (cx == ceil(s / tau)) return s;
    return tau * cx + y;
}

static double v_max(const chain_t *c, double tau)
{
    /* Q8: PAPER range [0, U(1,L) + sum C]; SAFE = 2(U(1,L)+sum C)+tau */
    if (c->v_range == VR_SAFE) return 2.0 * (c->Up[c->L] + c->SC) + tau;
    return c->Up[c->L] + c->SC;
}

typedef struct {
    int64_t g;  /* g(k,l,V) = ceil((V + U(k,l)) / tau) */
    int nf;     /* normal stage fits: M(k,l,g) <= M */
    int64_t d;  /* special memory shift ceil(M(k,l,g-1)(n_m-1)/M) (Q7) */
    int vn;     /* next delay level for k>1, or VN_OVERFLOW       (Q2, Q6, Q8) */
} trans_t;

static trans_t transition(const chain_t *c, double tau, double dV, int k, int l, int v)
{
    trans_t t;
    double V = (double)v * dV;
    double Ukl = U(c, k, l);
    t.g = (int64_t)ceil((V + Ukl) / tau);
    t.nf = Mem(c, k, l, t.g) <= c->M;
    int64_t D = Mem(c, k, l, t.g - 1);
    t.d = (D * (int64_t)(c->n_m - 1) + c->M - 1) / c->M;
    if (k > 1) {
        /* V' = (V (+) U(k,l)) (+) C(k-1)   (P:179 with reading Q2) */
        double Vn = oracle_oplus(oracle_oplus(V, Ukl, tau), c->C[k - 1], tau);
        double q = ceil(Vn / dV);
        if (q > (double)(c->n_v - 1))
            t.vn = (c->v_range == VR_SAFE) ? c->n_v - 1 : VN_OVERFLOW;
        else
            t.vn = (int)q;
    } else {
        t.vn = 0; /* unused: nothing precedes layer 1 (Q3) */
    }
    return t;
}

/* O5: smallest k in [1,l] with U(k,l) <= tau, or l+1 if none. */
static int kmin_of(const chain_t *c, double tau, int l)
{
    for (int k = 1; k <= l; k++)
        if (U(c, k, l) <= tau) return k;
    return l + 1;
}

#define IDX(c, l, p, v, m) \
    ((((size_t)(l) * (size_t)(c)->P + (size_t)(p)) * (size_t)(c)->n_v + (size_t)(v)) * (size_t)(c)->n_m + (size_t)(m))

/* ---------------------------------------------------------------- O6
 * Fill A[l][p][v][m] (and ARG if non-NULL) for one target period tau.
 * Recursion P:181-193 in decision form (Q1), base rows P:193 (Q10),
 * tie-break Q11, clamp Q12.  Returns the number of cell-updates. */
static int64_t fill_table(const chain_t *c, double tau, double *A, int32_t *ARG)
{
    const int L = c->L, P = c->P, n_v = c->n_v, n_m = c->n_m;
    const double dV = v_max(c, tau) / (double)(n_v - 1);
    int64_t updates = 0;

    for (int p = 0; p < P; p++)
        for (int v = 0; v < n_v; v++)
            for (int m = 0; m < n_m; m++) {
                A[IDX(c, 0, p, v, m)] = 0.0;          /* T(0,p,t_P,...) = t_P */
                if (ARG) ARG[IDX(c, 0, p, v, m)] = -1;
            }

    for (int l = 1; l <= L; l++) {
        double U1l = U(c, 1, l);
        /* p = 0: all of 1..l on the special processor (Q10) */
        for (int v = 0; v < n_v; v++) {
            trans_t t = transition(c, tau, dV, 1, l, v);
            for (int m = 0; m < n_m; m++) {
                int ok = (U1l <= tau) && ((int64_t)m + t.d <= (int64_t)(n_m - 1));
                A[IDX(c, l, 0, v, m)] = ok ? U1l : INFINITY;
                if (ARG) ARG[IDX(c, l, 0, v, m)] = ok ? 3 /* = 2*1 + S */ : -1;
            }
        }
        int kmin = kmin_of(c, tau, l);
        if (P > 1 && kmin <= l)
            updates += (int64_t)(l - kmin + 1) * (P - 1) * n_v * n_m;
        /* For each delay level v, the options k = kmin..l are scanned in
         * ascending order (N before S) for every cell (p, m) of the row; the
         * transition of (k, l, v) does not depend on (p, m), so it is computed
         * once per k.  Each cell still sees its options in the order of O6. */
        for (int v = 0; v < n_v; v++) {
            for (int p = 1; p < P; p++)
                for (int m = 0; m < n_m; m++) {
                    A[IDX(c, l, p, v, m)] = INFINITY;
                    if (ARG) ARG[IDX(c, l, p, v, m)] = -1;
                }
            for (int k = kmin; k <= l; k++) {
                trans_t t = transition(c, tau, dV, k, l, v);
                if (k > 1 && (t.vn == VN_OVERFLOW || c->C[k - 1] > tau)) continue;
                double Ukl = U(c, k, l);
                for (int p = 1; p < P; p++) {
                    for (int m = 0; m < n_m; m++) {
                        double *best = &A[IDX(c, l, p, v, m)];
                        /* T_N: stage k..l on a normal processor */
                        if (t.nf) {
                            double cand = A[IDX(c, k - 1, p - 1, t.vn, m)];
                            if (cand < *best) { *best = cand; if (ARG) ARG[IDX(c, l, p, v, m)] = 2 * k; }
                        }
                        /* T_S: stage k..l on the special processor */
                        if ((int64_t)m + t.d <= (int64_t)(n_m - 1)) {
                            double cand = Ukl + A[IDX(c, k - 1, p, t.vn, m + (int)t.d)];
                            if (cand <= tau && cand < *best) { *best = cand; if (ARG) ARG[IDX(c, l, p, v, m)] = 2 * k + 1; }
                        }
                    }
                }
            }
        }
    }
    return updates;
}

/* ---------------------------------------------------------------- O3 */
static double tau_of(const chain_t *c, int j, int n_c)
{
    double lb = c->Up[c->L] / (double)c->P;          /* Alg. 1 line 1 */
    double ub = c->Up[c->L] + c->SC;                  /* Alg. 1 line 2 (Q4) */
    if (n_c == 1) return ub;
    return lb + (double)j * ((ub - lb) / (double)(n_c - 1));   /* Q14 */
}

/* ---------------------------------------------------------------- O8/O9
 * Trace back the decisions from (L, P-1, v=0, m=0). */
static int traceback(const chain_t *c, double tau, const double *A, const int32_t *ARG,
                     int *n_stages, int *first, int *last, int *proc, double *load_period)
{
    (void)A;
    const double dV = v_max(c, tau) / (double)(c->n_v - 1);
    int l = c->L, p = c->P - 1, v = 0, m = 0, ns = 0;
    int *kind = (int *)malloc(sizeof(int) * (size_t)c->L);
    if (!kind) return OR_ENOMEM;
    while (l > 0) {
        if (p == 0) {
            first[ns] = 1; last[ns] = l; kind[ns] = 1; ns++;
            break;
        }
        int32_t arg = ARG[IDX(c, l, p, v, m)];
        if (arg < 0) { free(kind); return OR_EINVAL; } /* traceback from an infeasible cell */
        int k = arg >> 1, o = arg & 1;
        trans_t t = transition(c, tau, dV, k, l, v);
        first[ns] = k; last[ns] = l; kind[ns] = o; ns++;
        if (o) m += (int)t.d; else p -= 1;
        v = t.vn;
        l = k - 1;
    }
    /* reverse into chain order; number normal stages 0,1,.. ; special = P-1 */
    for (int i = 0; i < ns / 2; i++) {
        int j = ns - 1 - i, tmp;
        tmp = first[i]; first[i] = first[j]; first[j] = tmp;
        tmp = last[i]; last[i] = last[j]; last[j] = tmp;
        tmp = kind[i]; kind[i] = kind[j]; kind[j] = tmp;
    }
    int next_normal = 0;
    double lp = 0.0;
    for (int i = 0; i < ns; i++) {
        proc[i] = kind[i] ? c->P - 1 : next_normal++;
        if (!kind[i]) { double u = U(c, first[i], last[i]); if (u > lp) lp = u; }
        if (first[i] > 1 && c->C[first[i] - 1] > lp) lp = c->C[first[i] - 1];
    }
    *n_stages = ns;
    *load_period = lp;   /* the special load is max'ed in by the caller (O9) */
    free(kind);
    return OR_OK;
}

/* ====================================================================
 * Exported entry points (ctypes).
 * ==================================================================== */

/* Raw transition for unit tests: writes g, nf, d, vn. */
int oracle_transition(int L, const double *uF, const double *uB, const int64_t *W,
                      const int64_t *a, int P, int64_t M, double beta, int n_m, int n_v,
                      int v_range, double tau, int k, int l, int v,
                      int64_t *g, int *nf, int64_t *d, int *vn)
{
    chain_t c;
    int rc = chain_init(&c, L, uF, uB, W, a, P, M, beta, n_m, n_v, v_range);
    if (rc) { chain_free(&c); return rc; }
    if (k < 1 || k > l || l > L || v < 0 || v >= n_v) { chain_free(&c); return OR_EINVAL; }
    double dV = v_max(&c, tau) / (double)(n_v - 1);
    trans_t t = transition(&c, tau, dV, k, l, v);
    *g = t.g; *nf = t.nf; *d = t.d; *vn = t.vn;
    chain_free(&c);
    return OR_OK;
}

/* Prefix sums, C, lb, ub (O1, O3) for unit tests. */
int oracle_prep(int L, const double *uF, const double *uB, const int64_t *W, const int64_t *a,
                int P, double beta, double *Up, int64_t *Wp, int64_t *Ap, double *C,
                double *SC, double *lb, double *ub)
{
    chain_t c;
    int rc = chain_init(&c, L, uF, uB, W, a, P, 1, beta, 2, 2, VR_PAPER);
    if (rc) { chain_free(&c); return rc; }
    memcpy(Up, c.Up, sizeof(double) * (size_t)(L + 1));
    memcpy(Wp, c.Wp, sizeof(int64_t) * (size_t)(L + 1));
    memcpy(Ap, c.Ap, sizeof(int64_t) * (size_t)(L + 1));
    memcpy(C, c.C, sizeof(double) * (size_t)(L + 1));
    *SC = c.SC;
    *lb = tau_of(&c, 0, 2);
    *ub = tau_of(&c, 1, 1);
    chain_free(&c);
    return OR_OK;
}

int64_t oracle_mem(int L, const int64_t *W, const int64_t *a, int k, int l, int64_t g)
{
    chain_t c;
    double *u = (double *)malloc(sizeof(double) * (size_t)L);
    for (int i = 0; i < L; i++) u[i] = 1.0;
    chain_init(&c, L, u, u, W, a, 1, 1, 1.0, 2, 2, VR_PAPER);
    int64_t r = Mem(&c, k, l, g);
    chain_free(&c);
    free(u);
    return r;
}

/* Full DP table at a given tau: A_out[(L+1)*P*n_v*n_m] in [l][p][v][m] order,
 * arg_out (same shape, may be NULL) = 2k+o (o=1 special), -1 = infeasible. */
int oracle_table(int L, const double *uF, const double *uB, const int64_t *W, const int64_t *a,
                 int P, int64_t M, double beta, int n_m, int n_v, int v_range, double tau,
                 double *A_out, int32_t *arg_out, int64_t *cell_updates)
{
    chain_t c;
    int rc = chain_init(&c, L, uF, uB, W, a, P, M, beta, n_m, n_v, v_range);
    if (rc) { chain_free(&c); return rc; }
    if (!(tau > 0.0)) { chain_free(&c); return OR_EINVAL; }
    int64_t u = fill_table(&c, tau, A_out, arg_out);
    if (cell_updates) *cell_updates = u;
    chain_free(&c);
    return OR_OK;
}

/* Candidate sweep + winner + traceback (O3-O9).
 *   j_lo..j_hi-1  : candidate indices evaluated (j_hi<=n_c); all if j_lo=0,j_hi=n_c
 *   early_exit    : stop at the first feasible candidate (ascending j)
 *   tau_out[n_c]  : every candidate's period (always filled)
 *   root_out[n_c] : root value A_j[L][P-1][0][0] for evaluated j, NaN otherwise
 *   n_threads     : OpenMP threads over candidates (<=0: default)
 * Returns OR_OK, OR_INFEASIBLE (no evaluated candidate feasible) or an error. */
int oracle_solve(int L, const double *uF, const double *uB, const int64_t *W, const int64_t *a,
                 int P, int64_t M, double beta, int n_m, int n_v, int v_range,
                 int n_c, int j_lo, int j_hi, int early_exit, int n_threads,
                 double *tau_out, double *root_out,
                 double *period, double *load_period, double *special_load, int *cand_index,
                 int *n_stages, int *stage_first, int *stage_last, int *stage_proc,
                 int64_t *cell_updates)
{
    chain_t c;
    int rc = chain_init(&c, L, uF, uB, W, a, P, M, beta, n_m, n_v, v_range);
    if (rc || n_c < 1 || j_lo < 0 || j_hi > n_c || j_lo >= j_hi) {
        chain_free(&c);
        return rc ? rc : OR_EINVAL;
    }
    for (int j = 0; j < n_c; j++) { tau_out[j] = tau_of(&c, j, n_c); root_out[j] = NAN; }
    size_t cells = (size_t)(L + 1) * (size_t)P * (size_t)n_v * (size_t)n_m;
    int64_t total_updates = 0;
    int nt = 1;
#ifdef _OPENMP
    nt = n_threads > 0 ? n_threads : omp_get_max_threads();
#else
    (void)n_threads;
#endif
    int found = -1;
    /* candidates are processed in rounds of nt (one per thread); with early_exit
     * the scan stops after the first round that contains a feasible one. */
    double **tabs = (double **)calloc((size_t)nt, sizeof(double *));
    for (int t = 0; t < nt; t++) {
        tabs[t] = (double *)malloc(sizeof(double) * cells);
        if (!tabs[t]) { for (int u = 0; u < t; u++) free(tabs[u]); free(tabs); chain_free(&c); return OR_ENOMEM; }
    }
    for (int j0 = j_lo; j0 < j_hi && found < 0; j0 += nt) {
        int j1 = j0 + nt < j_hi ? j0 + nt : j_hi;
        int64_t round_updates = 0;
#ifdef _OPENMP
#pragma omp parallel for num_threads(nt) schedule(static, 1) reduction(+ : round_updates)
#endif
        for (int j = j0; j < j1; j++) {
            int t = 0;
#ifdef _OPENMP
            t = omp_get_thread_num();
#endif
            double tau = tau_out[j];
            round_updates += fill_table(&c, tau, tabs[t], NULL);
            root_out[j] = tabs[t][IDX(&c, L, P - 1, 0, 0)];
        }
        total_updates += round_updates;
        if (early_exit) {
            for (int j = j0; j < j1; j++)
                if (root_out[j] <= tau_out[j]) { found = j; break; }
        }
    }
    for (int t = 0; t < nt; t++) free(tabs[t]);
    free(tabs);
    if (found < 0)
        for (int j = j_lo; j < j_hi; j++)
            if (!isnan(root_out[j]) && root_out[j] <= tau_out[j]) { found = j; break; }  /* O7 */
    *cell_updates = total_updates;
    if (found < 0) {
        *period = INFINITY; *load_period = INFINITY; *special_load = INFINITY;
        *cand_index = -1; *n_stages = 0;
        chain_free(&c);
        return OR_INFEASIBLE;
    }
    /* re-solve the winner with decisions recorded, then trace back (O8) */
    double *A = (double *)malloc(sizeof(double) * cells);
    int32_t *ARG = (int32_t *)malloc(sizeof(int32_t) * cells);
    if (!A || !ARG) { free(A); free(ARG); chain_free(&c); return OR_ENOMEM; }
    double tau = tau_out[found];
    fill_table(&c, tau, A, ARG);
    double lp = 0.0;
    rc = traceback(&c, tau, A, ARG, n_stages, stage_first, stage_last, stage_proc, &lp);
    double root = A[IDX(&c, L, P - 1, 0, 0)];
    free(A); free(ARG);
    if (rc) { chain_free(&c); return rc; }
    *period = tau;                                  /* Q16 / Alg. 1 step 5 */
    *special_load = root;
    *load_period = root > lp ? root : lp;           /* O9 */
    *cand_index = found;
    chain_free(&c);
    return OR_OK;
}

/* ====================================================================
 * NEXT row f1: the paper-literal MadPipe-DP and Algorithm 1.
 *
 * T(l, p, t_P, m_P, V) of P:173 as a period (optimisation form), with t_P a
 * discretised state (n_t values in [0, U(1,L)]), for a fixed target
 * T-hat that drives the 1F1B* memory estimate (g, (+)):
 *   N: max(U(k,l), C(k-1), T(k-1, p-1, t, m, v'))   if M(k,l,g) <= M
 *   S: max(t'dt, C(k-1), T(k-1, p, t', m+d, v'))    if m+d <= n_m-1
 *              with t' = t + ceil(U(k,l)/dt) (reading L1: each special stage's
 *              load is rounded up to the t grid), infeasible if t' > n_t-1
 *   T(0,p,t,..) = t dt;  T(l,0,t,m,v) = U(1,l) + t dt if m + d(1,l,v) <= n_m-1
 *   T = min over k of the above, tie-break Q11; root T(L,P-1,0,0,0).
 * No tau-window here: any k is allowed, the period just grows.
 * Layout A[l][p][t][v][m].
 * ==================================================================== */
#define LIDX(c, nt, l, p, t, v, m) \
    (((((size_t)(l) * (size_t)(c)->P + (size_t)(p)) * (size_t)(nt) + (size_t)(t)) * (size_t)(c)->n_v + \
      (size_t)(v)) * (size_t)(c)->n_m + (size_t)(m))

static double dmax(double a, double b) { return a > b ? a : b; }

static int64_t literal_fill(const chain_t *c, double That, int n_t, double *A, int32_t *ARG)
{
    const int L = c->L, P = c->P, n_v = c->n_v, n_m = c->n_m;
    const double dV = v_max(c, That) / (double)(n_v - 1);
    const double dt = c->Up[L] / (double)(n_t - 1);
    int64_t updates = 0;
    for (int p = 0; p < P; p++)
        for (int t = 0; t < n_t; t++)
            for (int v = 0; v < n_v; v++)
                for (int m = 0; m < n_m; m++) {
                    A[LIDX(c, n_t, 0, p, t, v, m)] = (double)t * dt;     /* T(0,p,t_P,..) = t_P */
                    if (ARG) ARG[LIDX(c, n_t, 0, p, t, v, m)] = -1;
                }
    for (int l = 1; l <= L; l++) {
        double U1l = U(c, 1, l);
        for (int v = 0; v < n_v; v++) {
            trans_t tb = transition(c, That, dV, 1, l, v);
            for (int t = 0; t < n_t; t++)
                for (int m = 0; m < n_m; m++) {
                    int ok = (int64_t)m + tb.d <= (int64_t)(n_m - 1);
                    A[LIDX(c, n_t, l, 0, t, v, m)] = ok ? U1l + (double)t * dt : INFINITY;
                    if (ARG) ARG[LIDX(c, n_t, l, 0, t, v, m)] = ok ? 3 : -1;
                }
        }
        if (P > 1) updates += (int64_t)l * (P - 1) * n_t * n_v * n_m;
        for (int v = 0; v < n_v; v++) {
            for (int p = 1; p < P; p++)
                for (int t = 0; t < n_t; t++)
                    for (int m = 0; m < n_m; m++) {
                        A[LIDX(c, n_t, l, p, t, v, m)] = INFINITY;
                        if (ARG) ARG[LIDX(c, n_t, l, p, t, v, m)] = -1;
                    }
            for (int k = 1; k <= l; k++) {
                trans_t tr = transition(c, That, dV, k, l, v);
                if (k > 1 && tr.vn == VN_OVERFLOW) continue;
                double Ukl = U(c, k, l);
                double Ck = k > 1 ? c->C[k - 1] : 0.0;
                int64_t dts = (int64_t)ceil(Ukl / dt);
                for (int p = 1; p < P; p++)
                    for (int t = 0; t < n_t; t++)
                        for (int m = 0; m < n_m; m++) {
                            double *best = &A[LIDX(c, n_t, l, p, t, v, m)];
                            if (tr.nf) {                                   /* T_N */
                                double cand = dmax(dmax(Ukl, Ck), A[LIDX(c, n_t, k - 1, p - 1, t, tr.vn, m)]);
                                if (cand < *best) { *best = cand; if (ARG) ARG[LIDX(c, n_t, l, p, t, v, m)] = 2 * k; }
                            }
                            if ((int64_t)m + tr.d <= (int64_t)(n_m - 1) && (int64_t)t + dts <= (int64_t)(n_t - 1)) {
                                int t2 = t + (int)dts;                     /* T_S */
                                double cand = dmax(dmax((double)t2 * dt, Ck),
                                                   A[LIDX(c, n_t, k - 1, p, t2, tr.vn, m + (int)tr.d)]);
                                if (cand < *best) { *best = cand; if (ARG) ARG[LIDX(c, n_t, l, p, t, v, m)] = 2 * k + 1; }
                            }
                        }
            }
        }
    }
    return updates;
}

int oracle_literal_table(int L, const double *uF, const double *uB, const int64_t *W, const int64_t *a,
                         int P, int64_t M, double beta, int n_m, int n_v, int n_t, double That,
                         double *A_out, int32_t *arg_out)
{
    chain_t c;
    int rc = chain_init(&c, L, uF, uB, W, a, P, M, beta, n_m, n_v, VR_PAPER);
    if (rc || n_t < 2 || !(That > 0.0)) { chain_free(&c); return rc ? rc : OR_EINVAL; }
    literal_fill(&c, That, n_t, A_out, arg_out);
    chain_free(&c);
    return OR_OK;
}

/* Algorithm 1 (reading Q15): K calls of the literal DP; returns the
 * best max(T_i, That_i), its index and allocation (traceback of that call). */
int oracle_literal_solve(int L, const double *uF, const double *uB, const int64_t *W, const int64_t *a,
                         int P, int64_t M, double beta, int n_m, int n_v, int n_t, int K,
                         double *T_hist, double *That_hist, double *period, int *best_iter,
                         int *n_stages, int *stage_first, int *stage_last, int *stage_proc)
{
    chain_t c;
    int rc = chain_init(&c, L, uF, uB, W, a, P, M, beta, n_m, n_v, VR_PAPER);
    if (rc || n_t < 2 || K < 1) { chain_free(&c); return rc ? rc : OR_EINVAL; }
    size_t cells = (size_t)(L + 1) * (size_t)P * (size_t)n_t * (size_t)n_v * (size_t)n_m;
    double *A = (double *)malloc(sizeof(double) * cells);
    int32_t *ARG = (int32_t *)malloc(sizeof(int32_t) * cells);
    if (!A || !ARG) { free(A); free(ARG); chain_free(&c); return OR_ENOMEM; }
    double lb = c.Up[L] / (double)P;                  /* line 1 */
    double ub = c.Up[L] + c.SC;                       /* line 2 (Q4) */
    double That = lb;                                 /* line 3 */
    double best = INFINITY;
    int bi = -1;
    for (int i = 0; i < K; i++) {
        literal_fill(&c, That, n_t, A, NULL);
        double T = A[LIDX(&c, n_t, L, P - 1, 0, 0, 0)];   /* T_i = MadPipe-DP(That_i) */
        T_hist[i] = T; That_hist[i] = That;
        double Tm = T > That ? T : That;                   /* max(T_i, That_i) */
        if (Tm < best) { best = Tm; bi = i; }
        double lo = T < That ? T : That;
        if (lo > lb) lb = lo;                              /* lb <- max(lb, min(T, That)) */
        if (Tm < ub) ub = Tm;                              /* ub <- min(ub, max(T, That)) */
        That = (lb + ub) / 2.0;
    }
    *period = best;
    *best_iter = bi;
    *n_stages = 0;
    if (bi >= 0 && isfinite(best)) {
        double Tb = That_hist[bi];
        literal_fill(&c, Tb, n_t, A, ARG);
        const double dV = v_max(&c, Tb) / (double)(n_v - 1);
        const double dt = c.Up[L] / (double)(n_t - 1);
        int l = L, p = P - 1, t = 0, v = 0, m = 0, ns = 0;
        int *kind = (int *)malloc(sizeof(int) * (size_t)L);
        while (l > 0) {
            if (p == 0) { stage_first[ns] = 1; stage_last[ns] = l; kind[ns] = 1; ns++; break; }
            int32_t arg = ARG[LIDX(&c, n_t, l, p, t, v, m)];
            if (arg < 0) break;
            int k = arg >> 1, o = arg & 1;
            trans_t tr = transition(&c, Tb, dV, k, l, v);
            stage_first[ns] = k; stage_last[ns] = l; kind[ns] = o; ns++;
            if (o) { m += (int)tr.d; t += (int)(int64_t)ceil(U(&c, k, l) / dt); } else p -= 1;
            v = tr.vn;
            l = k - 1;
        }
        for (int i = 0; i < ns / 2; i++) {
            int j = ns - 1 - i, tmp;
            tmp = stage_first[i]; stage_first[i] = stage_first[j]; stage_first[j] = tmp;
            tmp = stage_last[i]; stage_last[i] = stage_last[j]; stage_last[j] = tmp;
            tmp = kind[i]; kind[i] = kind[j]; kind[j] = tmp;
        }
        int next_normal = 0;
        for (int i = 0; i < ns; i++) stage_proc[i] = kind[i] ? P - 1 : next_normal++;
        *n_stages = ns;
        free(kind);
    }
    free(A); free(ARG);
    chain_free(&c);
    return isfinite(best) ? OR_OK : OR_INFEASIBLE;
}
