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
// M(k,l,g) of P:159: sum_{i=k..l}(3W_i + g a_{i-1}) + 2(a_{k-1} + a_l), the
// buffer terms dropped at k = 1 and l = L.
__device__ __forceinline__ int64_t mem_kl(const Job &J, int k, int l, int64_t g) {
    int64_t m = 3 * (J.Wp[l] - J.Wp[k - 1]) + g * (J.Ap[l] - J.Ap[k - 1]);
    if (k > 1) m += 2 * J.a[k - 1];
    if (l < J.L) m += 2 * J.a[l];
    return m;
}

// x (+) y of P:177.
__device__ __forceinline__ double oplus(double x, double y, double tau) {
    const double cx = ceil(__ddiv_rn(x, tau));
    const double s = __dadd_rn(x, y);
    if (cx == ceil(__ddiv_rn(s, tau))) return s;
    return __dadd_rn(__dmul_rn(tau, cx), y);
}

constexpr int32_t kSkip = (int32_t)0x80000000;

// d = ceil(D (n_m-1) / M) for D >= 0, M > 0 (reading Q7), exactly, without a
// software int64 division: an fp64 estimate, then a 128-bit check of
// (d-1) M < D (n_m-1) <= d M and a +-1 correction.  D (n_m-1) + M - 1 fits in
// int64 (madpipe_validate); only d <= n_m matters to the callers, larger values
// mean "does not fit", so the result is clamped to n_m+1.
__device__ __forceinline__ int64_t ceil_div_levels(int64_t D, int nm1, int64_t M) {
    const uint64_t X = (uint64_t)D * (uint64_t)nm1;
    if (X == 0) return 0;
    if (D > M) return nm1 + 2;                       // d > n_m - 1: no level fits
    int64_t d = (int64_t)ceil(__ddiv_rn((double)X, (double)M));
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

// Transition of stage k..l entered with delay level v:
// g = ceil((V + U(k,l)) / tau); nf = M(k,l,g) <= M; d = ceil(M(k,l,g-1)(n_m-1)/M)
// (reading Q7); for k > 1 the next delay V' = (V (+) U) (+) C(k-1) rounded up to
// the grid (readings Q2, Q6, Q8).  Returns kSkip if neither option is possible.
// skip_comm = false is the optimisation form of NEXT row f1 (mp_literal.cu),
// where a communication longer than T-hat is not a skip: it enters the max.
__device__ __forceinline__ int32_t transition(const Job &J, int k, int l, int v, double Ukl,
                                              int64_t *d_out, bool skip_comm = true) {
    const double V = __dmul_rn((double)v, J.dV);
    const int64_t g = (int64_t)ceil(__ddiv_rn(__dadd_rn(V, Ukl), J.tau));
    const bool nf = mem_kl(J, k, l, g) <= J.M;
    const int64_t D = mem_kl(J, k, l, g - 1);
    const int64_t d = ceil_div_levels(D, J.n_m - 1, J.M);
    if (d_out) *d_out = d;
    int vn = 0;
    if (k > 1) {
        const double ck = J.C[k - 1];
        if (skip_comm && ck > J.tau) return kSkip;
        const double Vn = oplus(oplus(V, Ukl, J.tau), ck, J.tau);
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
