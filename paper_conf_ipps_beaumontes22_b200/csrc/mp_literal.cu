// mp_literal.cu -- NEXT row f1: the paper-literal MadPipe-DP (optimisation form,
// P:173-193, with t_P discretised as in P:233) and Algorithm 1 (P:203-205,
// reading Q15) on the GPU.  This is the serial baseline the decision-form
// candidate sweep replaces: K dependent DP calls, each a
// wavefront over L layers.
//
// For a target T-hat (which drives g and (+) exactly as in the decision form):
//   T(l,p,t,m,v) = min over k of
//     N: max(U(k,l), C(k-1), T(k-1, p-1, t, m, v'))          if M(k,l,g) <= M
//     S: max(t' dt, C(k-1), T(k-1, p, t', m+d, v'))          if m+d <= n_m-1
//        t' = t + ceil(U(k,l)/dt) <= n_t-1 (reading L1)
//   T(0,p,t,..) = t dt;  T(l,0,t,m,v) = U(1,l) + t dt if m + d(1,l,v) <= n_m-1
// Layout per DP: A[l][v][t][p][NMP] (fp64).  Same operation order as the
// oracle's literal_fill (max / min are exact; t' dt is one rounded product).
#include <cmath>
#include <cstdint>
#include <cuda_runtime.h>

#include "mp_device.cuh"
#include "mp_internal.cuh"

namespace mp {

struct LitGeom {
    int n_t;
    double dt;       // U(1,L) / (n_t - 1)
};

__device__ __forceinline__ double dmax2(double a, double b) { return a > b ? a : b; }

__device__ __forceinline__ size_t lit_row(const Job &J, int n_t, int nmp, int l, int v, int t) {
    return ((((size_t)l * J.n_v + v) * n_t + t) * (size_t)J.P) * nmp;
}

__global__ void lit_init_kernel(const Job *job, LitGeom G, int nmp) {
    const Job &J = *job;
    const int64_t cells = (int64_t)J.n_v * G.n_t * J.P * nmp;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cells;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(i % nmp);
        const int t = (int)((i / ((int64_t)nmp * J.P)) % G.n_t);
        J.table[i] = m < J.n_m ? __dmul_rn((double)t, G.dt) : MP_INF;   // T(0,p,t_P,..) = t_P
    }
}

// one CTA per (v, chunk of (t, p) rows); thread per (t, p) row of NMP levels
template <int NMP>
__global__ void __launch_bounds__(256) lit_step_kernel(const Job *job, LitGeom G, int l) {
    __shared__ int32_t s_tr[512];
    __shared__ double s_U[512];
    __shared__ int32_t s_dt[512];
    const Job &J = *job;
    const int v = blockIdx.y;
    const int n_t = G.n_t;
    const int rows = n_t * J.P;
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    const double Ul = J.Up[l];
    const size_t rowlen = (size_t)J.P * NMP;
    double *out = J.table + lit_row(J, n_t, NMP, l, v, 0);
    const int kmin = kmin_mem(J, l);
    const int n_m = J.n_m;
    const int t = r / J.P, p = r - (r / J.P) * J.P;
    double best[NMP];
#pragma unroll
    for (int m = 0; m < NMP; m++) best[m] = MP_INF;
    if (r < rows && p == 0) {   // base row (reading Q10)
        int64_t d;
        const double U1l = __dsub_rn(Ul, J.Up[0]);
        (void)transition(J, 1, l, v, U1l, &d, false);
#pragma unroll
        for (int m = 0; m < NMP; m++)
            best[m] = (m < n_m && (int64_t)m + d <= (int64_t)(n_m - 1))
                          ? __dadd_rn(U1l, __dmul_rn((double)t, G.dt)) : MP_INF;
    }
    for (int kc0 = kmin; kc0 <= l; kc0 += 512) {
        const int nk = min(512, l + 1 - kc0);
        __syncthreads();
        for (int e = threadIdx.x; e < nk; e += blockDim.x) {
            const int k = kc0 + e;
            const double Ukl = __dsub_rn(Ul, J.Up[k - 1]);
            s_tr[e] = transition(J, k, l, v, Ukl, nullptr, false);
            s_U[e] = Ukl;
            s_dt[e] = (int32_t)ceil(__ddiv_rn(Ukl, G.dt));
        }
        __syncthreads();
        if (r >= rows || p == 0) continue;
        for (int e = 0; e < nk; e++) {
            const int32_t tr = s_tr[e];
            if (tr < 0) continue;
            const int k = kc0 + e;
            const int vn = tr & 0xFFFF, d = (tr >> 16) & 0xFF;
            const double Ck = k > 1 ? J.C[k - 1] : 0.0;
            const double Ukl = s_U[e];
            if (tr & (1 << 24)) {      // N
                const double *src = J.table + lit_row(J, n_t, NMP, k - 1, vn, t) + (size_t)(p - 1) * NMP;
                const double base = dmax2(Ukl, Ck);
#pragma unroll
                for (int m = 0; m < NMP; m++) {
                    const double c = dmax2(base, src[m]);
                    best[m] = c < best[m] ? c : best[m];
                }
            }
            const int t2 = t + s_dt[e];
            if (d <= n_m - 1 && t2 <= n_t - 1) {   // S
                const double *src = J.table + lit_row(J, n_t, NMP, k - 1, vn, t2) + (size_t)p * NMP + d;
                const double base = dmax2(__dmul_rn((double)t2, G.dt), Ck);
#pragma unroll
                for (int m = 0; m < NMP; m++) {
                    if (m + d <= n_m - 1) {
                        const double c = dmax2(base, src[m]);
                        best[m] = c < best[m] ? c : best[m];
                    }
                }
            }
        }
    }
    if (r < rows) {
        double *o = out + (size_t)t * rowlen + (size_t)p * NMP;
#pragma unroll
        for (int m = 0; m < NMP; m++) o[m] = m < n_m ? best[m] : MP_INF;
    }
}

// decision of one cell: smallest 2k+o whose candidate equals the cell (Q11)
__device__ int lit_code(const Job &J, LitGeom G, int nmp, int l, int p, int t, int v, int m, double cell,
                        int k_begin, int k_step) {
    const double Ul = J.Up[l];
    int code = 0x7fffffff;
    for (int k = k_begin; k <= l; k += k_step) {
        const double Ukl = __dsub_rn(Ul, J.Up[k - 1]);
        int64_t d;
        const int32_t tr = transition(J, k, l, v, Ukl, &d, false);
        if (tr < 0) continue;
        const int vn = tr & 0xFFFF;
        const double Ck = k > 1 ? J.C[k - 1] : 0.0;
        if ((tr & (1 << 24)) &&
            dmax2(dmax2(Ukl, Ck), J.table[lit_row(J, G.n_t, nmp, k - 1, vn, t) + (size_t)(p - 1) * nmp + m]) == cell) {
            code = 2 * k;
            break;
        }
        const int t2 = t + (int)ceil(__ddiv_rn(Ukl, G.dt));
        if ((int64_t)m + d <= (int64_t)(J.n_m - 1) && t2 <= G.n_t - 1 &&
            dmax2(dmax2(__dmul_rn((double)t2, G.dt), Ck),
                  J.table[lit_row(J, G.n_t, nmp, k - 1, vn, t2) + (size_t)p * nmp + m + d]) == cell) {
            code = 2 * k + 1;
            break;
        }
    }
    return code;
}

__global__ void lit_export_kernel(const Job *job, LitGeom G, int nmp, double *A_out, int32_t *arg_out) {
    // output layout [l][p][t][v][m] (the oracle's)
    const Job &J = *job;
    const int n_t = G.n_t, n_v = J.n_v, n_m = J.n_m, P = J.P;
    const int64_t cells = (int64_t)(J.L + 1) * P * n_t * n_v * n_m;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cells;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(i % n_m);
        const int v = (int)((i / n_m) % n_v);
        const int t = (int)((i / ((int64_t)n_m * n_v)) % n_t);
        const int p = (int)((i / ((int64_t)n_m * n_v * n_t)) % P);
        const int l = (int)(i / ((int64_t)n_m * n_v * n_t * P));
        const double cell = J.table[lit_row(J, n_t, nmp, l, v, t) + (size_t)p * nmp + m];
        A_out[i] = cell;
        if (arg_out) {
            int code = -1;
            if (l > 0 && cell < MP_INF) {
                if (p == 0) code = 3;
                else {
                    const int c = lit_code(J, G, nmp, l, p, t, v, m, cell, kmin_mem(J, l), 1);
                    code = c == 0x7fffffff ? -2 : c;
                }
            }
            arg_out[i] = code;
        }
    }
}

// traceback from (L, P-1, t=0, v=0, m=0): stages (first, last, kind) reversed
__global__ void lit_traceback_kernel(const Job *job, LitGeom G, int nmp, int32_t *stages, int32_t *n_out) {
    const Job &J = *job;
    __shared__ int s_code[32];
    __shared__ int s_l, s_p, s_t, s_v, s_m, s_ns, s_done;
    int32_t *first = stages, *last = stages + J.L, *kind = stages + 2 * J.L;
    if (threadIdx.x == 0) { s_l = J.L; s_p = J.P - 1; s_t = 0; s_v = 0; s_m = 0; s_ns = 0; s_done = 0; }
    __syncthreads();
    while (true) {
        __syncthreads();
        const int l = s_l, p = s_p, t = s_t, v = s_v, m = s_m;
        if (l == 0 || s_done) break;
        if (p == 0) {
            __syncthreads();   // every thread has read s_l before thread 0 overwrites it (p is block-uniform)
            if (threadIdx.x == 0) { first[s_ns] = 1; last[s_ns] = l; kind[s_ns] = 1; s_ns++; s_l = 0; }
            continue;
        }
        const double cell = J.table[lit_row(J, G.n_t, nmp, l, v, t) + (size_t)p * nmp + m];
        int code = cell < MP_INF ? lit_code(J, G, nmp, l, p, t, v, m, cell, kmin_mem(J, l) + threadIdx.x,
                                            blockDim.x)
                                 : 0x7fffffff;
        for (int o = 16; o > 0; o >>= 1) code = min(code, __shfl_xor_sync(0xffffffffu, code, o));
        if ((threadIdx.x & 31) == 0) s_code[threadIdx.x >> 5] = code;
        __syncthreads();
        if (threadIdx.x == 0) {
            int c = 0x7fffffff;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) c = min(c, s_code[w]);
            if (c == 0x7fffffff) {
                s_done = 1;
            } else {
                const int k = c >> 1, o = c & 1;
                int64_t d;
                const double Ukl = __dsub_rn(J.Up[l], J.Up[k - 1]);
                const int32_t tr = transition(J, k, l, v, Ukl, &d, false);
                first[s_ns] = k; last[s_ns] = l; kind[s_ns] = o; s_ns++;
                if (o) { s_m = m + (int)d; s_t = t + (int)ceil(__ddiv_rn(Ukl, G.dt)); } else s_p = p - 1;
                s_v = tr & 0xFFFF;
                s_l = k - 1;
            }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) *n_out = s_done ? -s_ns - 1 : s_ns;
}

void launch_lit_init(const Job *job, int n_t, double dt, int nmp, int64_t cells, cudaStream_t s) {
    LitGeom G{n_t, dt};
    int g = (int)std::min<int64_t>(4096, (cells + 255) / 256);
    lit_init_kernel<<<g, 256, 0, s>>>(job, G, nmp);
}

void launch_lit_step(const Job *job, int n_t, double dt, int nmp, int n_v, int P, int l, cudaStream_t s) {
    LitGeom G{n_t, dt};
    const dim3 grid((n_t * P + 255) / 256, n_v);
    switch (nmp) {
    case 2: lit_step_kernel<2><<<grid, 256, 0, s>>>(job, G, l); break;
    case 4: lit_step_kernel<4><<<grid, 256, 0, s>>>(job, G, l); break;
    case 8: lit_step_kernel<8><<<grid, 256, 0, s>>>(job, G, l); break;
    case 16: lit_step_kernel<16><<<grid, 256, 0, s>>>(job, G, l); break;
    case 32: lit_step_kernel<32><<<grid, 256, 0, s>>>(job, G, l); break;
    default: lit_step_kernel<64><<<grid, 256, 0, s>>>(job, G, l); break;
    }
}

void launch_lit_export(const Job *job, int n_t, double dt, int nmp, double *A_out, int32_t *arg_out,
                       cudaStream_t s) {
    LitGeom G{n_t, dt};
    lit_export_kernel<<<512, 256, 0, s>>>(job, G, nmp, A_out, arg_out);
}

void launch_lit_traceback(const Job *job, int n_t, double dt, int nmp, int32_t *stages, int32_t *n_out,
                          cudaStream_t s) {
    LitGeom G{n_t, dt};
    lit_traceback_kernel<<<1, 256, 0, s>>>(job, G, nmp, stages, n_out);
}

}  // namespace mp
