// mp_kernels.cu -- sm_100a kernels of the MadPipe-DP hot path.
//
// All fp64 arithmetic goes through __dadd_rn / __dsub_rn / __dmul_rn /
// __ddiv_rn (and the file is compiled with --fmad=false) so that no FMA
// contraction can change a rounding: results are bit-identical to the plain
// CPU oracle.  "P:n" = line n of the MadPipe paper text; "Qn", "On" = DESIGN.md
// readings / normative steps.
#include <cstdint>
#include <cuda_runtime.h>
#include <math_constants.h>

#include "mp_internal.cuh"
#include "mp_device.cuh"

namespace mp {


// ---------------------------------------------------------------------------
// a1: profile prep (P:155 U, P:159 sums of W and a_{i-1}, P:147 C = 2a/beta,
// P:205 lines 1-2 lb/ub with reading Q4).  One CTA per chain; the prefix sums
// are sequential (one thread) so the rounding order is the textbook one (Q13).
// ---------------------------------------------------------------------------
__global__ void prep_kernel(ChainDev *chains) {
    ChainDev &c = chains[blockIdx.x];
    const int L = c.L;
    constexpr int CH = 1024;
    __shared__ double s_u[CH];
    __shared__ int64_t s_w[CH];
    __shared__ int64_t s_a[CH];
    __shared__ double s_up;
    __shared__ int64_t s_wp, s_ap;
    if (threadIdx.x == 0) {
        s_up = 0.0; s_wp = 0; s_ap = 0;
        c.Up[0] = 0.0; c.Wp[0] = 0; c.Ap[0] = 0; c.C[0] = 0.0;
    }
    for (int base = 1; base <= L; base += CH) {
        const int n = min(CH, L - base + 1);
        __syncthreads();
        for (int t = threadIdx.x; t < n; t += blockDim.x) {
            const int i = base + t;                       // layer i (1-based)
            s_u[t] = __dadd_rn(c.uF[i - 1], c.uB[i - 1]); // uF_i + uB_i
            s_w[t] = c.W[i - 1];
            s_a[t] = c.a[i - 1];                          // a_{i-1}
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            double up = s_up;
            int64_t wp = s_wp, ap = s_ap;
            for (int t = 0; t < n; t++) {
                up = __dadd_rn(up, s_u[t]);
                wp += s_w[t];
                ap += s_a[t];
                c.Up[base + t] = up; c.Wp[base + t] = wp; c.Ap[base + t] = ap;
            }
            s_up = up; s_wp = wp; s_ap = ap;
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double sc = 0.0;
        for (int i = 1; i <= L - 1; i++) {
            const double ci = __ddiv_rn(__dmul_rn(2.0, (double)c.a[i]), c.beta);
            c.C[i] = ci;
            sc = __dadd_rn(sc, ci);
        }
        c.C[L] = 0.0;
        const double U = c.Up[L];
        c.scal[0] = sc;
        c.scal[1] = __ddiv_rn(U, (double)c.P);   // lb
        c.scal[2] = __dadd_rn(U, sc);            // ub
        c.scal[3] = U;
    }
}

void launch_prep(ChainDev *chains_dev, int n_chains, cudaStream_t s) {
    prep_kernel<<<n_chains, 256, 0, s>>>(chains_dev);
}

// ---------------------------------------------------------------------------
// a2: candidate grid (reading Q14) and the delay grid (reading Q8).
// ---------------------------------------------------------------------------
__global__ void jobs_init_kernel(Job *jobs, int n_jobs) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_jobs) return;
    Job &J = jobs[i];
    const double sc = J.scal[0], lb = J.scal[1], ub = J.scal[2], U = J.scal[3];
    double tau;
    if (J.n_c == 1)
        tau = ub;
    else
        tau = __dadd_rn(lb, __dmul_rn((double)J.j, __ddiv_rn(__dsub_rn(ub, lb), (double)(J.n_c - 1))));
    const double vmax = J.vsafe ? __dadd_rn(__dmul_rn(2.0, __dadd_rn(U, sc)), tau) : __dadd_rn(U, sc);
    J.tau = tau;
    J.dV = __ddiv_rn(vmax, (double)(J.n_v - 1));
}

void launch_jobs_init(Job *jobs, int n_jobs, cudaStream_t s) {
    jobs_init_kernel<<<(n_jobs + 127) / 128, 128, 0, s>>>(jobs, n_jobs);
}

// ---------------------------------------------------------------------------
// Slab l = 0: A[0][v][p][m] = 0 (T(0,p,t_P,..) = t_P), padding = +inf.
// ---------------------------------------------------------------------------
__global__ void init_slab0_kernel(const Job *jobs, int nmp) {
    const Job &J = jobs[blockIdx.y];
    const int64_t cells = (int64_t)J.n_v * J.P * nmp;
    if (J.rowflag)
        for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < J.n_v; v += gridDim.x * blockDim.x)
            J.rowflag[v] = 1u;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cells;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(i % nmp);
        J.table[i] = m < J.n_m ? 0.0 : MP_INF;
    }
}

void launch_init_slab0(const Job *jobs, int n_jobs, int nmp, int max_cells, cudaStream_t s) {
    int bx = (max_cells + 255) / 256;
    if (bx > 64) bx = 64;
    init_slab0_kernel<<<dim3(bx, n_jobs), 256, 0, s>>>(jobs, nmp);
}

// ---------------------------------------------------------------------------
// a4 + a5: one wavefront step for layer l over every job of the batch.
//
// A[l][v][p][m] = min over k in [kmin(l), l] of
//     N: A[k-1][vn][p-1][m]                      if nf
//     S: U(k,l) + A[k-1][vn][p][m+d]             if m+d <= n_m-1, <= tau
// then clamped: values > tau become +inf (reading Q12; min and clamp commute).
// p = 0 is the base row.  A CTA owns vb delay rows x np processor rows
// of one job; each thread owns one (v, p) row of NMP memory levels in registers.
// Transitions of a chunk of k are staged in shared memory (a3, fused).
// ---------------------------------------------------------------------------
template <int NMP>
__global__ void __launch_bounds__(kThreads) step_kernel(const Job *__restrict__ jobs,
                                                        const int32_t *__restrict__ tile_job,
                                                        int l) {
    __shared__ Job sJ;
    __shared__ int32_t s_tr[kTransSmem];
    __shared__ double s_U[kMaxKChunk];
    const int tid = threadIdx.x;
    const int jid = tile_job[blockIdx.x];
    if (tid == 0) sJ = jobs[jid];
    __syncthreads();
    const Job &J = sJ;
    if (l > J.L) return;
    const int t = blockIdx.x - J.tile0;
    const int vt = t / J.n_ptiles, pt = t % J.n_ptiles;
    const int v0 = vt * J.vb;
    const int vcount = min(J.vb, J.n_v - v0);
    const int p_lo = 1 + pt * J.np;
    const int np = max(0, min(J.np, J.P - p_lo));
    const size_t rowlen = (size_t)J.P * NMP;
    const size_t slab = (size_t)J.n_v * rowlen;
    double *__restrict__ out = J.table + (size_t)l * slab;
    const double tau = J.tau;
    const double Ul = J.Up[l];
    const int n_m = J.n_m;

    // base row p = 0: layers 1..l all on the special GPU (reading Q10)
    if (pt == 0 && tid < vcount) {
        const int v = v0 + tid;
        const double U1l = __dsub_rn(Ul, J.Up[0]);
        int64_t d;
        (void)transition(J, 1, l, v, U1l, &d);
        double *o = out + (size_t)v * rowlen;
#pragma unroll
        for (int m = 0; m < NMP; m++)
            o[m] = (m < n_m && U1l <= tau && (int64_t)m + d <= (int64_t)(n_m - 1)) ? U1l : MP_INF;
    }
    if (np <= 0) return;

    const int kmin = max(kmin_of(J, l), kmin_mem(J, l));
    const int pairs = vcount * np;
    const bool active = tid < pairs;
    const int vv = active ? tid / np : 0;
    const int pp = p_lo + (active ? tid % np : 0);
    double best[NMP];
#pragma unroll
    for (int m = 0; m < NMP; m++) best[m] = MP_INF;

    const double *__restrict__ tab = J.table;
    const int kc_len = min(kMaxKChunk, kTransSmem / vcount);
    for (int kc0 = kmin; kc0 <= l; kc0 += kc_len) {
        const int nk = min(kc_len, l + 1 - kc0);
        __syncthreads();
        unsigned live = 0;
        for (int e = tid; e < nk * vcount; e += blockDim.x) {
            const int kk = e / vcount, v2 = e - kk * vcount;
            const int k = kc0 + kk;
            const double Ukl = __dsub_rn(Ul, J.Up[k - 1]);
            const int32_t tr = transition(J, k, l, v0 + v2, Ukl, nullptr);
            s_tr[e] = tr;
            live += tr >= 0;
            if (v2 == 0) s_U[kk] = Ukl;
        }
        if (pt == 0) {   // count each live (k, l, v) once: it feeds (P-1) n_m relaxations
            for (int o = 16; o > 0; o >>= 1) live += __shfl_xor_sync(0xffffffffu, live, o);
            if ((tid & 31) == 0 && live)
                atomicAdd(J.eff, (unsigned long long)live * (unsigned long long)(J.P - 1) *
                                     (unsigned long long)n_m);
        }
        __syncthreads();
        if (!active) continue;
        for (int kk = 0; kk < nk; kk++) {
            const int32_t tr = s_tr[kk * vcount + vv];
            if (tr < 0) continue;
            const int vn = tr & 0xFFFF;
            const int d = (tr >> 16) & 0xFF;
            const double *row = tab + (size_t)(kc0 + kk - 1) * slab + (size_t)vn * rowlen;
            if (tr & (1 << 24)) {   // N: stage k..l on a normal GPU
                const double2 *src = reinterpret_cast<const double2 *>(row + (size_t)(pp - 1) * NMP);
#pragma unroll
                for (int h = 0; h < NMP / 2; h++) {
                    const double2 x = __ldg(src + h);
                    best[2 * h] = x.x < best[2 * h] ? x.x : best[2 * h];
                    best[2 * h + 1] = x.y < best[2 * h + 1] ? x.y : best[2 * h + 1];
                }
            }
            if (d <= n_m - 1) {     // S: stage k..l on the special GPU
                const double U = s_U[kk];
                const double *src = row + (size_t)pp * NMP + d;
#pragma unroll
                for (int m = 0; m < NMP; m++) {
                    if (m + d <= n_m - 1) {
                        const double c = __dadd_rn(U, __ldg(src + m));
                        best[m] = c < best[m] ? c : best[m];
                    }
                }
            }
        }
    }
    if (active) {
        double2 *o = reinterpret_cast<double2 *>(out + (size_t)(v0 + vv) * rowlen + (size_t)pp * NMP);
#pragma unroll
        for (int h = 0; h < NMP / 2; h++) {
            double2 r;
            r.x = (2 * h < n_m && best[2 * h] <= tau) ? best[2 * h] : MP_INF;
            r.y = (2 * h + 1 < n_m && best[2 * h + 1] <= tau) ? best[2 * h + 1] : MP_INF;
            o[h] = r;
        }
    }
}

void launch_step(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp, int threads,
                 cudaStream_t s) {
    switch (nmp) {
    case 2: step_kernel<2><<<n_tiles, threads, 0, s>>>(jobs, tile_job, l); break;
    case 4: step_kernel<4><<<n_tiles, threads, 0, s>>>(jobs, tile_job, l); break;
    case 8: step_kernel<8><<<n_tiles, threads, 0, s>>>(jobs, tile_job, l); break;
    case 16: step_kernel<16><<<n_tiles, threads, 0, s>>>(jobs, tile_job, l); break;
    case 32: step_kernel<32><<<n_tiles, threads, 0, s>>>(jobs, tile_job, l); break;
    default: step_kernel<64><<<n_tiles, threads, 0, s>>>(jobs, tile_job, l); break;
    }
}

// ---------------------------------------------------------------------------
// a3 (+ a4) for the persistent step kernel, computed by all SMs in parallel
// (one warp per (job, delay row v)) instead of inside the step kernel's producer:
// the base row A[l][v][0][*], and the list of USEFUL transitions of row
// v in ascending k over the window [max(kmin_tau, kmin_W), l]:
// live and with a source row A[k-1][v'] that holds a finite value
// (a row that is +inf everywhere can only contribute +inf).  Also counts the
// job's effective and useful relaxations.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(64) trans_kernel(const Job *jobs, int l, int nmp, size_t buf_off,
                                                   int verify_last) {
    // one half-warp per delay row v of the job (4 rows per 64-thread CTA: small
    // CTAs so that one fits on an SM beside the two resident step-kernel CTAs -- this
    // kernel runs on a second stream, overlapped with the step kernel of layer l-1);
    // the job descriptor is read once into shared memory.  buf_off selects the list
    // buffer of layer l (double-buffered).  verify_last = 0: the source row of k = l
    // (slab l-1) may still be being written by the concurrent step kernel, so its
    // flag is not consulted -- that entry is kept (and counted as read).
    __shared__ Job sJ;
    if (threadIdx.x < sizeof(Job) / 8)
        reinterpret_cast<uint64_t *>(&sJ)[threadIdx.x] =
            __ldg(reinterpret_cast<const uint64_t *>(jobs + blockIdx.y) + threadIdx.x);
    __syncthreads();
    const Job &J = sJ;
    if (l > J.L) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int half = lane >> 4, hl = lane & 15;
    const int v = blockIdx.x * 4 + warp * 2 + half;
    const bool row_ok = v < J.n_v;
    if (__ballot_sync(0xffffffffu, row_ok) == 0u) return;
    const size_t rowlen = (size_t)J.P * nmp;
    const double Ul = J.Up[l];
    // base row p = 0 (reading Q10), and the row flag of (l, v): it is reset
    // here and OR-ed by the step kernel for p >= 1
    if (row_ok) {
        const double U1l = __dsub_rn(Ul, J.Up[0]);
        int64_t d;
        (void)transition(J, 1, l, v, U1l, &d);
        const bool ok = U1l <= J.tau && d <= (int64_t)(J.n_m - 1);
        double *o = J.table + (size_t)l * J.n_v * rowlen + (size_t)v * rowlen;
        for (int m = hl; m < nmp; m += 16)
            o[m] = (m < J.n_m && U1l <= J.tau && (int64_t)m + d <= (int64_t)(J.n_m - 1)) ? U1l : MP_INF;
        if (hl == 0) J.rowflag[(size_t)l * J.n_v + v] = ok ? 1u : 0u;
    }
    const int kmin = J.kwin[l];   // max(kmin_tau(l), kmin_W(l)), precomputed by window_kernel
    unsigned live = 0, useful = 0;
    int n = 0;
    TransEntry *list = J.tlist + buf_off + (size_t)(row_ok ? v : 0) * J.code_cap;
    const RowCtx rc = row_ctx(J, row_ok ? v : 0);
    for (int kb = kmin; kb <= l; kb += 16) {   // same trip count in both halves (same job, layer)
        const int k = kb + hl;
        int32_t tr = -1;
        double Ukl = 0.0;
        bool use = false;
        if (row_ok && k <= l) {
            Ukl = __dsub_rn(Ul, J.Up[k - 1]);
            tr = transition_rc(J, k, l, rc, Ukl, nullptr);
            if (tr >= 0) {
                live++;
                // a source row that is +inf everywhere can only contribute +inf (exact skip)
                use = (k == l && !verify_last) || J.rowflag[(size_t)(k - 1) * J.n_v + (tr & 0xFFFF)] != 0u;
                useful += use;
            }
        }
        const unsigned bal = (__ballot_sync(0xffffffffu, use) >> (half * 16)) & 0xFFFFu;
        if (use) {
            TransEntry e;
            e.U = Ukl; e.code = tr; e.k = k;
            list[n + __popc(bal & ((1u << hl) - 1u))] = e;
        }
        n += __popc(bal);
    }
    if (row_ok && hl == 0) J.tcount[buf_off / J.code_cap + v] = n;
    for (int o = 16; o > 0; o >>= 1) {
        live += __shfl_xor_sync(0xffffffffu, live, o);
        useful += __shfl_xor_sync(0xffffffffu, useful, o);
    }
    if (lane == 0 && live && J.P > 1) {
        const unsigned long long per = (unsigned long long)(J.P - 1) * (unsigned long long)J.n_m;
        atomicAdd(J.eff, (unsigned long long)live * per);
        if (useful) atomicAdd(J.useful, (unsigned long long)useful * per);
    }
}

// window start of every layer of every job (the binary searches are the same for
// all delay rows of a job, so they run once per batch instead of once per row)
__global__ void window_kernel(const Job *jobs, int n_jobs, int max_L) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const int job = i / max_L, l = 1 + i - (i / max_L) * max_L;
    if (job >= n_jobs) return;
    const Job &J = jobs[job];
    if (l > J.L) return;
    J.kwin[l] = max(kmin_of(J, l), kmin_mem(J, l));
}

void launch_window(const Job *jobs, int n_jobs, int max_L, cudaStream_t s) {
    const int n = n_jobs * max_L;
    window_kernel<<<(n + 255) / 256, 256, 0, s>>>(jobs, n_jobs, max_L);
}

void launch_trans(const Job *jobs, int n_jobs, int n_v_max, int l, int nmp, size_t buf_off, int verify_last,
                  cudaStream_t s) {
    trans_kernel<<<dim3((n_v_max + 3) / 4, n_jobs), 64, 0, s>>>(jobs, l, nmp, buf_off, verify_last);
}

// ---------------------------------------------------------------------------
// a6: root test.  feasible_j = A_j[L][P-1][0][0] <= tau_j (O7); the smallest
// feasible j of each chain is kept with atomicMin.
// ---------------------------------------------------------------------------
__global__ void root_kernel(const Job *jobs, int n_jobs, int nmp, int32_t *jl_per_chain,
                            double *root_out, double *tau_out) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_jobs) return;
    const Job &J = jobs[i];
    const size_t rowlen = (size_t)J.P * nmp;
    const size_t slab = (size_t)J.n_v * rowlen;
    const double r = J.table[(size_t)J.L * slab + (size_t)(J.P - 1) * nmp];
    if (root_out) root_out[J.gid] = r;
    if (tau_out) tau_out[J.gid] = J.tau;
    if (r <= J.tau) atomicMin(jl_per_chain + J.chain, J.j);
}

void launch_root(const Job *jobs, int n_jobs, int nmp, int32_t *jl_per_chain, double *root_out,
                 double *tau_out, cudaStream_t s) {
    root_kernel<<<(n_jobs + 127) / 128, 128, 0, s>>>(jobs, n_jobs, nmp, jl_per_chain, root_out,
                                                     tau_out);
}

// Exact relaxation count of each job.
__global__ void count_kernel(const Job *jobs, int n_jobs, unsigned long long *counts) {
    const Job &J = jobs[blockIdx.x];
    if (J.P < 2) return;
    unsigned long long acc = 0;
    for (int l = 1 + threadIdx.x; l <= J.L; l += blockDim.x) {
        const int km = kmin_of(J, l);
        if (km <= l) acc += (unsigned long long)(l - km + 1);
    }
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0 && acc)
        atomicAdd(counts + blockIdx.x,
                  acc * (unsigned long long)(J.P - 1) * (unsigned long long)J.n_v * (unsigned long long)J.n_m);
}

void launch_count(const Job *jobs, int n_jobs, unsigned long long *counts, cudaStream_t s) {
    count_kernel<<<n_jobs, 128, 0, s>>>(jobs, n_jobs, counts);
}

// ---------------------------------------------------------------------------
// Decision of one cell: the smallest code 2k+o whose candidate value equals the
// cell's value (tie-break Q11).  Same candidate arithmetic as step_kernel.
// ---------------------------------------------------------------------------
__device__ int cell_code_partial(const Job &J, int nmp, int l, int p, int v, int m, double cell,
                                 int k_begin, int k_step) {
    const size_t rowlen = (size_t)J.P * nmp;
    const size_t slab = (size_t)J.n_v * rowlen;
    const double Ul = J.Up[l];
    int code = 0x7fffffff;
    for (int k = k_begin; k <= l; k += k_step) {
        const double Ukl = __dsub_rn(Ul, J.Up[k - 1]);
        if (Ukl > J.tau) continue;
        int64_t d;
        const int32_t tr = transition(J, k, l, v, Ukl, &d);
        if (tr < 0) continue;
        const int vn = tr & 0xFFFF;
        const double *row = J.table + (size_t)(k - 1) * slab + (size_t)vn * rowlen;
        if ((tr & (1 << 24)) && row[(size_t)(p - 1) * nmp + m] == cell) { code = 2 * k; break; }
        if ((int64_t)m + d <= (int64_t)(J.n_m - 1)) {
            const double c = __dadd_rn(Ukl, row[(size_t)p * nmp + m + d]);
            if (c <= J.tau && c == cell) { code = 2 * k + 1; break; }
        }
    }
    return code;
}

// ---------------------------------------------------------------------------
// a8: device traceback (O8/O9).  One CTA per job.  Stages are written
// in chain order with processors numbered (normal 0,1,.. in chain order,
// special P-1), plus the allocation's load period.
// ---------------------------------------------------------------------------
__global__ void traceback_kernel(const Job *jobs, int nmp, TraceOut *outs, int32_t *stages,
                                 int stage_stride) {
    const Job &J = jobs[blockIdx.x];
    TraceOut &T = outs[blockIdx.x];
    int32_t *first = stages + (size_t)blockIdx.x * 3 * stage_stride;
    int32_t *last = first + stage_stride;
    int32_t *proc = last + stage_stride;
    __shared__ int s_code[32];
    __shared__ int s_l, s_p, s_v, s_m, s_ns, s_done;
    const size_t rowlen = (size_t)J.P * nmp;
    const size_t slab = (size_t)J.n_v * rowlen;
    const double root = J.table[(size_t)J.L * slab + (size_t)(J.P - 1) * nmp];
    if (threadIdx.x == 0) {
        s_l = J.L; s_p = J.P - 1; s_v = 0; s_m = 0; s_ns = 0; s_done = 0;
        T.status = (root <= J.tau) ? 0 : 1;
    }
    __syncthreads();
    if (!(root <= J.tau)) {
        if (threadIdx.x == 0) { T.n_stages = 0; T.load_period = MP_INF; T.special_load = MP_INF; }
        return;
    }
    while (true) {
        __syncthreads();
        const int l = s_l, p = s_p, v = s_v, m = s_m;
        if (l == 0 || s_done) break;
        if (p == 0) {   // base case: stage 1..l on the special GPU
            __syncthreads();   // every thread has read s_l before thread 0 overwrites it (p is block-uniform)
            if (threadIdx.x == 0) {
                first[s_ns] = 1; last[s_ns] = l; proc[s_ns] = -1; s_ns++;
                s_l = 0;
            }
            continue;
        }
        const double cell = J.table[(size_t)l * slab + (size_t)v * rowlen + (size_t)p * nmp + m];
        const int km = max(kmin_of(J, l), kmin_mem(J, l));
        int code = cell_code_partial(J, nmp, l, p, v, m, cell, km + threadIdx.x, blockDim.x);
        for (int o = 16; o > 0; o >>= 1) code = min(code, __shfl_xor_sync(0xffffffffu, code, o));
        if ((threadIdx.x & 31) == 0) s_code[threadIdx.x >> 5] = code;
        __syncthreads();
        if (threadIdx.x == 0) {
            int c = 0x7fffffff;
            for (int w = 0; w < (int)(blockDim.x >> 5); w++) c = min(c, s_code[w]);
            if (c == 0x7fffffff) {
                s_done = 1; T.status = 2;
            } else {
                const int k = c >> 1, o = c & 1;
                int64_t d;
                const int32_t tr = transition(J, k, l, v, __dsub_rn(J.Up[l], J.Up[k - 1]), &d);
                first[s_ns] = k; last[s_ns] = l; proc[s_ns] = o ? -1 : -2; s_ns++;
                if (o) s_m = m + (int)d; else s_p = p - 1;
                s_v = tr & 0xFFFF;
                s_l = k - 1;
            }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const int ns = s_ns;
        for (int i = 0; i < ns / 2; i++) {   // reverse into chain order
            const int j = ns - 1 - i;
            int t;
            t = first[i]; first[i] = first[j]; first[j] = t;
            t = last[i]; last[i] = last[j]; last[j] = t;
            t = proc[i]; proc[i] = proc[j]; proc[j] = t;
        }
        int next_normal = 0;
        double lp = 0.0;
        for (int i = 0; i < ns; i++) {
            if (proc[i] == -2) {
                proc[i] = next_normal++;
                const double u = __dsub_rn(J.Up[last[i]], J.Up[first[i] - 1]);
                if (u > lp) lp = u;
            } else {
                proc[i] = J.P - 1;
            }
            if (first[i] > 1 && J.C[first[i] - 1] > lp) lp = J.C[first[i] - 1];
        }
        T.n_stages = ns;
        T.special_load = root;
        T.load_period = root > lp ? root : lp;
    }
}

void launch_traceback(const Job *jobs, int n_jobs, int nmp, TraceOut *outs, int32_t *stages,
                      int stage_stride, cudaStream_t s) {
    traceback_kernel<<<n_jobs, 256, 0, s>>>(jobs, nmp, outs, stages, stage_stride);
}

// Decision table export (parity tests): thread per cell (l >= 1).
__global__ void argmin_kernel(const Job *job, int nmp, int32_t *arg_out, int L, int P, int n_v,
                              int n_m) {
    const Job &J = *job;
    const int64_t cells = (int64_t)(L + 1) * P * n_v * n_m;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cells;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(i % n_m);
        const int v = (int)((i / n_m) % n_v);
        const int p = (int)((i / ((int64_t)n_m * n_v)) % P);
        const int l = (int)(i / ((int64_t)n_m * n_v * P));
        const size_t rowlen = (size_t)P * nmp;
        const size_t slab = (size_t)n_v * rowlen;
        const double cell = J.table[(size_t)l * slab + (size_t)v * rowlen + (size_t)p * nmp + m];
        int code = -1;
        if (l > 0 && cell <= J.tau) {
            if (p == 0) {
                code = 3;
            } else {
                const int c = cell_code_partial(J, nmp, l, p, v, m, cell,
                                                max(kmin_of(J, l), kmin_mem(J, l)), 1);
                code = c == 0x7fffffff ? -2 : c;
            }
        }
        arg_out[i] = code;
    }
}

void launch_argmin(const Job *job, int nmp, int32_t *arg_out, int L, int P, int n_v, int n_m,
                   cudaStream_t s) {
    argmin_kernel<<<256, 256, 0, s>>>(job, nmp, arg_out, L, P, n_v, n_m);
}

// Table export in the oracle's [l][p][v][m] order (parity tests).
__global__ void export_kernel(const Job *job, int nmp, double *A_out, int L, int P, int n_v,
                              int n_m) {
    const Job &J = *job;
    const int64_t cells = (int64_t)(L + 1) * P * n_v * n_m;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cells;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int m = (int)(i % n_m);
        const int v = (int)((i / n_m) % n_v);
        const int p = (int)((i / ((int64_t)n_m * n_v)) % P);
        const int l = (int)(i / ((int64_t)n_m * n_v * P));
        const size_t rowlen = (size_t)P * nmp;
        const size_t slab = (size_t)n_v * rowlen;
        A_out[i] = J.table[(size_t)l * slab + (size_t)v * rowlen + (size_t)p * nmp + m];
    }
}

void launch_export(const Job *job, int nmp, double *A_out, int L, int P, int n_v, int n_m,
                   cudaStream_t s) {
    export_kernel<<<256, 256, 0, s>>>(job, nmp, A_out, L, P, n_v, n_m);
}

}  // namespace mp
