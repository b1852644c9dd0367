// mp_device.cuh -- device helpers shared by every kernel that evaluates a DP
// transition, so that all of them use the identical fp64 operation sequence.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <math_constants.h>

#include "mp_internal.cuh"

namespace mp {

#define MP_INF CUDART_INF

// ---------------------------------------------------------------------------
// Device helpers: memory model, (+), transition (a3).
// ---------------------------------------------------------------------------
constexpr int32_t kSkip = (int32_t)0x80000000;

// d = ceil(D (n_m-1) / M) for D >= 0, M > 0 (reading Q7), exactly, without a
// software int64 division: an fp64 estimate (D (n_m-1) times the job's 1/M), then a
// 128-bit check of (d-1) M < D (n_m-1) <= d M and a +-1 correction.  D (n_m-1) + M - 1
// fits in int64 (madpipe_validate); only d <= n_m matters to the callers, larger
// values mean "does not fit", so the result is clamped to n_m+1.
__device__ __forceinline__ int64_t ceil_div_levels(int64_t D, int nm1, int64_t M, double invM) {
    const uint64_t X = (uint64_t)D * (uint64_t)nm1;
    if (X == 0) return 0;
    if (D > M) return nm1 + 2;                       // d > n_m - 1: no level fits
    int64_t d = (int64_t)ceil((double)X * invM);
    if (d < 1) d = 1;
    // d*M >= X ?  (128-bit: d <= n_m+1 is small, M < 2^63)
    auto ge = [&](int64_t q) {
        const uint64_t lo = (uint64_t)q * (uint64_t)M;
        const uint64_t hi = __umul64hi((uint64_t)q, (uint64_t)M);
        return hi > 0 || lo >= X;
    };
    while (!ge(d)) d++;
    while (d > 1 && ge(d - 1)) d--;
    return d;
}

// What a transition needs of its delay row v alone (hoisted out of k-loops):
// V = v dV, ceil(V / tau) (the first ceiling of V (+) U) and 1/M.
struct RowCtx {
    double V, cxV, invM;
};
__device__ __forceinline__ RowCtx row_ctx(const Job &J, int v) {
    RowCtx r;
    r.V = __dmul_rn((double)v, J.dV);
    r.cxV = ceil(__ddiv_rn(r.V, J.tau));
    r.invM = 1.0 / (double)J.M;
    return r;
}

// Transition of stage k..l entered with delay level v:
// g = ceil((V + U(k,l)) / tau); nf = M(k,l,g) <= M; d = ceil(M(k,l,g-1)(n_m-1)/M)
// (reading Q7); for k > 1 the next delay V' = (V (+) U) (+) C(k-1) rounded up to
// the grid (readings Q2, Q6, Q8).  Returns kSkip if neither option is possible.
// skip_comm = false is the optimisation form of NEXT row f1 (mp_literal.cu),
// where a communication longer than T-hat is not a skip: it enters the max.
// Definitions followed (the oracle's operation sequence):
//   M(k,l,g) = sum_{i=k..l}(3W_i + g a_{i-1}) + 2(a_{k-1} + a_l), the buffer terms
//              dropped at k = 1 and l = L, in int64;
//   x (+) y  = x + y if ceil(x/tau) = ceil((x+y)/tau), else tau ceil(x/tau) + y.
// The quotient (V + U) / tau serves both g and V (+) U, and M(k,l,g-1) is M(k,l,g)
// minus sum a_{i-1} (the same int64 value), so every result is bit-identical.
__device__ __forceinline__ int32_t transition_rc(const Job &J, int k, int l, const RowCtx &rc, double Ukl,
                                                 int64_t *d_out, bool skip_comm = true) {
    const double s = __dadd_rn(rc.V, Ukl);
    const double cs = ceil(__ddiv_rn(s, J.tau));
    const int64_t g = (int64_t)cs;
    const int64_t dA = J.Ap[l] - J.Ap[k - 1];
    int64_t base = 3 * (J.Wp[l] - J.Wp[k - 1]);
    if (k > 1) base += 2 * J.a[k - 1];
    if (l < J.L) base += 2 * J.a[l];
    const int64_t Mg = base + g * dA;                // M(k,l,g)
    const bool nf = Mg <= J.M;
    const int64_t d = ceil_div_levels(Mg - dA, J.n_m - 1, J.M, rc.invM);
    if (d_out) *d_out = d;
    int vn = 0;
    if (k > 1) {
        const double ck = J.C[k - 1];
        if (skip_comm && ck > J.tau) return kSkip;
        // x1 = V (+) U: ceil(V/tau) vs ceil((V+U)/tau) = cs
        const bool same = rc.cxV == cs;
        const double x1 = same ? s : __dadd_rn(__dmul_rn(J.tau, rc.cxV), Ukl);
        // x1 (+) C(k-1): ceil(x1/tau) is cs when x1 = V+U
        const double cx1 = same ? cs : ceil(__ddiv_rn(x1, J.tau));
        const double s2 = __dadd_rn(x1, ck);
        const double Vn = cx1 == ceil(__ddiv_rn(s2, J.tau)) ? s2 : __dadd_rn(__dmul_rn(J.tau, cx1), ck);
        const double q = ceil(__ddiv_rn(Vn, J.dV));
        if (q > (double)(J.n_v - 1)) {
            if (!J.vsafe) return kSkip;
            vn = J.n_v - 1;
        } else {
            vn = (int)q;
        }
    }
    if (!nf && d > (int64_t)(J.n_m - 1)) return kSkip;
    return pack_trans(vn, d, nf);
}

__device__ __forceinline__ int32_t transition(const Job &J, int k, int l, int v, double Ukl,
                                              int64_t *d_out, bool skip_comm = true) {
    return transition_rc(J, k, l, row_ctx(J, v), Ukl, d_out, skip_comm);
}

// smallest k in [1,l] with U(k,l) = Up[l] - Up[k-1] <= tau (O5); l+1 if none.
// U(k,l) is non-increasing in k (monotone rounding), so bisection is exact.
__device__ __forceinline__ int kmin_of(const Job &J, int l) {
    const double Ul = J.Up[l];
    if (__dsub_rn(Ul, J.Up[l - 1]) > J.tau) return l + 1;
    int lo = 1, hi = l;   // answer in [lo, hi]
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (__dsub_rn(Ul, J.Up[mid - 1]) <= J.tau) hi = mid; else lo = mid + 1;
    }
    return lo;
}

// Smallest k in [1,l] whose weights alone fit: 3 (Wp[l] - Wp[k-1]) <= M; l+1 if
// none.  For k below it, M(k,l,g) >= 3 sum W > M for every g >= 0, so neither a
// normal GPU nor the special one (M(k,l,g-1) with g >= 1) can
// take stage k..l: transition() would return kSkip.  Pruning these k is exact.
__device__ __forceinline__ int kmin_mem(const Job &J, int l) {
    const int64_t Wl = J.Wp[l];
    if (3 * (Wl - J.Wp[l - 1]) > J.M) return l + 1;
    int lo = 1, hi = l;
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (3 * (Wl - J.Wp[mid - 1]) <= J.M) hi = mid; else lo = mid + 1;
    }
    return lo;
}

}  // namespace mp
