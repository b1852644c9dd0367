// mp_step_persist.cu -- the wavefront min-plus step (a4-a5) as a persistent,
// warp-specialised, TMA-pipelined sm_100a kernel (the default step kernel).
//
// Same recursion as step_kernel (mp_kernels.cu), P:181-193 in decision form (Q1):
//   A[l][v][p][m] = clamp_tau( min over live k of
//        N: A[k-1][v'][p-1][m]            (normal GPU fits)
//        S: U(k,l) + A[k-1][v'][p][m+d]   (special GPU) ).
// The transitions (k, v) -> (v', nf, d) of layer l were computed beforehand by
// trans_kernel (a3) into J.codes, for the window starting at *J.kmin_l.
//
// Structure:
//   * grid = resident CTAs (1-2 per SM); CTA c takes tiles c, c+G, c+2G, ...
//     A tile is vb delay rows x np processor rows of one job.
//   * warp 8 is the producer.  Per tile it writes the base row p = 0 (a4),
//     reads the window's codes (32 at a time, one coalesced load per lane),
//     compacts the k with a live row (ballot), and for each such k streams the
//     source row segments A[k-1][v'][p_lo-1 .. p_lo+np-1][*] of the live delay
//     rows into a `nst`-stage shared-memory ring with cp.async.bulk, each stage
//     completing on its mbarrier.  Up to nst lanes issue stages concurrently.
//   * warps 0-7 are consumers.  ROW mode (NMP <= 16): a thread owns one
//     (v, p) row of NMP levels as NMP/2 16-byte chunks held in a lane-rotated
//     order, which makes every quarter-warp's 16-byte shared loads hit 8
//     distinct bank groups while register indices stay compile-time.  PAIR mode
//     (NMP >= 32): a thread owns one (v, p, m-pair).  Either way the shift d is
//     uniform per warp.  At the tile's last stage they clamp to tau and store.
// min is exact and order-free, so results equal the oracle's bit for bit.
#include <cstdint>
#include <cuda_runtime.h>

#include "mp_device.cuh"
#include "mp_internal.cuh"

namespace mp {

namespace {

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar)
        : "memory");
}
__device__ __forceinline__ double dmin(double a, double b) { return b < a ? b : a; }

}  // namespace

constexpr int kNstMax = 12;          // ring stages (runtime nst <= kNstMax)
constexpr int kPCons = 256;          // consumer threads (8 warps); + 1 producer warp
constexpr int kMaxVb = 8;            // delay rows per tile
constexpr int kMaxGroups = 128;      // live k collected per producer round

// per-stage metadata written by the producer, read by the consumers
struct StageMeta {
    double *out;              // output of row v0, processor p_lo (row v0+vv at out + vv*rowlen)
    double tau;
    double U;                 // U(k,l) of the stage's k
    int32_t tr[kMaxVb];       // transition code per delay row (<0: not live)
    uint32_t *flag;           // row flags of (l, v0): row v0+vv at flag[vv]
    int32_t rowlen;           // P*NMP
    int16_t np, vcount, n_m, flags;   // flags: 1 = last stage of the tile, 2 = no data, 4 = terminate
};

template <int NMP>
__global__ void __launch_bounds__(kPCons + 32, 2) step_persist_kernel(const Job *__restrict__ jobs,
                                                                      const int32_t *__restrict__ tile_job,
                                                                      int n_tiles, int l, int stage_doubles,
                                                                      int nst) {
    constexpr int C = NMP / 2;                       // 16-byte chunks per processor row
    constexpr bool ROW = NMP <= 16;
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ __align__(8) uint64_t full[kNstMax];
    __shared__ __align__(8) uint64_t empty[kNstMax];
    __shared__ StageMeta meta[kNstMax];
    __shared__ Job pJ;                               // producer's copy of the current tile's job
    __shared__ int32_t p_tr[kMaxGroups * kMaxVb];    // live codes of the round's groups
    __shared__ int32_t p_grp[kMaxGroups];            // k of each group
    __shared__ double p_U[kMaxGroups];               // U(k,l) of each group

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const uint32_t full0 = smem_u32(&full[0]), empty0 = smem_u32(&empty[0]);
    const uint32_t ring_s = smem_u32(dsm);
    if (tid == 0) {
        for (int s = 0; s < nst; s++) {
            mbar_init(full0 + 8 * s, 1);
            mbar_init(empty0 + 8 * s, kPCons / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const double *ring = reinterpret_cast<const double *>(dsm);

    if (warp == kPCons / 32) {
        // ======================================================= producer warp
        int gi = 0;              // stages issued so far
        int slot0 = 0, use0 = 0; // slot of stage gi and how many times that slot was used before
        for (int tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
            const int jid = tile_job[tile];
            __syncwarp();
            {   // cooperative copy of the job descriptor (one 8-byte word per lane)
                static_assert(sizeof(Job) % 8 == 0 && sizeof(Job) <= 32 * 8 * 2, "Job size");
                const uint64_t *src = reinterpret_cast<const uint64_t *>(jobs + jid);
                uint64_t *dst = reinterpret_cast<uint64_t *>(&pJ);
                for (int w = lane; w < (int)(sizeof(Job) / 8); w += 32) dst[w] = __ldg(src + w);
            }
            __syncwarp();
            const Job &J = pJ;
            if (l > J.L) continue;
            const int t = tile - J.tile0;
            const int vt = t / J.n_ptiles, pt = t - (t / J.n_ptiles) * J.n_ptiles;
            const int v0 = vt * J.vb;
            const int vcount = min(J.vb, J.n_v - v0);
            const int p_lo = 1 + pt * J.np;
            const int np = max(0, min(J.np, J.P - p_lo));
            const size_t rowlen = (size_t)J.P * NMP;
            const size_t slab = (size_t)J.n_v * rowlen;
            const int seg_doubles = (np + 1) * NMP;
            const uint32_t seg_bytes = (uint32_t)seg_doubles * 8u;
            double *out = J.table + (size_t)l * slab;
            const double Ul = J.Up[l];
            const double tau = J.tau;
            const int n_m = J.n_m;
            if (pt == 0 && lane < vcount) {          // base row p = 0 (Q10)
                const int v = v0 + lane;
                const double U1l = __dsub_rn(Ul, J.Up[0]);
                int64_t d;
                (void)transition(J, 1, l, v, U1l, &d);
                double *o = out + (size_t)v * rowlen;
#pragma unroll
                for (int m = 0; m < NMP; m++)
                    o[m] = (m < n_m && U1l <= tau && (int64_t)m + d <= (int64_t)(n_m - 1)) ? U1l : MP_INF;
                if (U1l <= tau && d <= (int64_t)(n_m - 1)) atomicOr(J.rowflag + (size_t)l * J.n_v + v, 1u);
            }
            if (np <= 0) continue;
            const int kmin = *J.kmin_l;
            const int per = 32 / vcount;              // k per pass (vcount <= 8)
            const int kk = lane / vcount, v2 = lane - kk * vcount;
            const unsigned grp_mask = ((1u << vcount) - 1u) << (kk * vcount);
            const int32_t *codes = J.codes + (size_t)(v0 + v2) * J.code_cap;
            double *tile_out = out + (size_t)v0 * rowlen + (size_t)p_lo * NMP;
            uint32_t *tile_flag = J.rowflag + (size_t)l * J.n_v + v0;
            auto fill_meta = [&](StageMeta &M, int flags) {
                M.out = tile_out; M.tau = tau; M.rowlen = (int32_t)rowlen; M.flag = tile_flag;
                M.np = (int16_t)np; M.vcount = (int16_t)vcount; M.n_m = (int16_t)n_m;
                M.flags = (int16_t)flags;
            };
            bool closed = false;
            for (int kb = kmin; kb <= l;) {
                // ---- collect up to kMaxGroups live groups (k with >= 1 live delay row)
                int ngrp = 0;
                for (; kb <= l && ngrp + per <= kMaxGroups; kb += per) {
                    const int k = kb + kk;
                    const bool valid = kk < per && k <= l;
                    const int32_t tr = valid ? __ldg(codes + (k - kmin)) : -1;
                    const double Ukl = (valid && v2 == 0) ? __dsub_rn(Ul, __ldg(J.Up + k - 1)) : 0.0;
                    const unsigned live = __ballot_sync(0xffffffffu, tr >= 0);
                    const bool leader = valid && (v2 == 0) && (live & grp_mask);
                    const unsigned leaders = __ballot_sync(0xffffffffu, leader);
                    const int rank = ngrp + __popc(leaders & ((1u << lane) - 1u));
                    const int myrank = __shfl_sync(0xffffffffu, rank, valid ? kk * vcount : 0);
                    if (valid && (live & grp_mask)) {
                        p_tr[myrank * kMaxVb + v2] = tr;
                        if (v2 == 0) { p_grp[myrank] = k; p_U[myrank] = Ukl; }
                    }
                    ngrp += __popc(leaders);
                }
                const bool done = kb > l;
                __syncwarp();
                // ---- one stage per live group, in rounds of at most nst stages: the slots
                // of a round are distinct, so each lane's parity wait refers to the previous
                // use of its own slot (never two phases ahead, where mbarrier parity aliases)
                for (int g0 = 0; g0 < ngrp; g0 += nst) {
                    const int g = g0 + lane;
                    if (lane < nst && g < ngrp) {
                        // stage gi+g -> slot and use count, without runtime division: the
                        // round holds < nst stages, so the slot wraps at most once
                        int s = slot0 + lane, use = use0;
                        if (s >= nst) { s -= nst; use++; }
                        if (use > 0) mbar_wait(empty0 + 8 * s, (uint32_t)((use - 1) & 1));
                        const int k = p_grp[g];
                        const double *src = J.table + (size_t)(k - 1) * slab + (size_t)(p_lo - 1) * NMP;
                        uint32_t bytes = 0;
                        StageMeta &M = meta[s];
                        for (int w = 0; w < kMaxVb; w++) {   // copies first, metadata after
                            const int32_t trw = w < vcount ? p_tr[g * kMaxVb + w] : -1;
                            M.tr[w] = trw;
                            if (trw < 0) continue;
                            bytes += seg_bytes;
                            bulk_g2s(ring_s + 8u * (uint32_t)(s * stage_doubles + w * seg_doubles),
                                     src + (size_t)(trw & 0xFFFF) * rowlen, seg_bytes, full0 + 8 * s);
                        }
                        fill_meta(M, done && g == ngrp - 1 ? 1 : 0);
                        M.U = p_U[g];
                        mbar_arrive_expect_tx(full0 + 8 * s, bytes);
                    }
                    __syncwarp();
                    const int adv = min(nst, ngrp - g0);   // stages issued in this round
                    slot0 += adv;
                    if (slot0 >= nst) { slot0 -= nst; use0++; }
                }
                gi += ngrp;
                if (done) { closed = ngrp > 0; break; }
            }
            if (!closed) {   // no live stage at the end of the window: close with an empty stage
                if (lane == 0) {
                    if (use0 > 0) mbar_wait(empty0 + 8 * slot0, (uint32_t)((use0 - 1) & 1));
                    fill_meta(meta[slot0], 1 | 2);
                    mbar_arrive(full0 + 8 * slot0);
                }
                gi += 1;
                if (++slot0 == nst) { slot0 = 0; use0++; }
            }
        }
        __syncwarp();
        if (lane == 0) {
            if (use0 > 0) mbar_wait(empty0 + 8 * slot0, (uint32_t)((use0 - 1) & 1));
            meta[slot0].flags = 4;
            mbar_arrive(full0 + 8 * slot0);
        }
        return;
    }

    // =========================================================== consumer warps
    constexpr int NB = ROW ? NMP : 2;   // accumulators per thread
    double best[NB];
#pragma unroll
    for (int i = 0; i < NB; i++) best[i] = MP_INF;
    int cur_np = -1, cur_vc = -1, vv = 0, pp_off = 0, h = 0, rot = 0;
    bool active = false;
    int s = 0, phase = 0;
    for (;; ) {
        mbar_wait(full0 + 8 * s, (uint32_t)phase);
        const StageMeta &M = meta[s];
        const int flags = M.flags;
        if (flags & 4) break;
        const int np = M.np, vcount = M.vcount, n_m = M.n_m;
        if (np != cur_np || vcount != cur_vc) {
            if (ROW) {
                const int rowgroup = ((np + 31) / 32) * 32;
                vv = tid / rowgroup;
                pp_off = tid - vv * rowgroup;
                // lane rotation of the chunks: 8 consecutive threads of a quarter-warp
                // start at 8 distinct 16-byte bank groups
                constexpr int G8 = C >= 8 ? 1 : 8 / C;
                constexpr int RM = C >= 8 ? 8 : C;
                rot = (pp_off / G8) % RM;
                active = vv < vcount && pp_off < np;
            } else {
                const int rowgroup = ((np * C + 31) / 32) * 32;
                vv = tid / rowgroup;
                const int q = tid - vv * rowgroup;
                pp_off = q / C;
                h = q - pp_off * C;
                active = vv < vcount && pp_off < np;
            }
            cur_np = np; cur_vc = vcount;
        }
        if (!(flags & 2) && active) {
            const int32_t tr = M.tr[vv];
            if (tr >= 0) {
                const double *seg = ring + (size_t)s * stage_doubles + (size_t)vv * (np + 1) * NMP;
                const double *rowN = seg + pp_off * NMP;           // processor p-1
                const double *rowS = rowN + NMP;                    // processor p
                const int d = (tr >> 16) & 0xFF;
                const double U = M.U;
                if (ROW) {
                    if (tr & (1 << 24)) {                           // N
#pragma unroll
                        for (int c = 0; c < C; c++) {
                            const int j = (c + rot) & (C - 1);
                            const double2 x = *reinterpret_cast<const double2 *>(rowN + 2 * j);
                            best[2 * c] = dmin(best[2 * c], x.x);
                            best[2 * c + 1] = dmin(best[2 * c + 1], x.y);
                        }
                    }
                    if (d <= n_m - 1) {                             // S
                        if ((d & 1) == 0) {
                            const int e = d >> 1;
#pragma unroll
                            for (int c = 0; c < C; c++) {
                                const int j = (c + rot) & (C - 1);
                                if (2 * j + d <= n_m - 1) {
                                    const double2 y = *reinterpret_cast<const double2 *>(rowS + 2 * (j + e));
                                    best[2 * c] = dmin(best[2 * c], __dadd_rn(U, y.x));
                                    if (2 * j + 1 + d <= n_m - 1)
                                        best[2 * c + 1] = dmin(best[2 * c + 1], __dadd_rn(U, y.y));
                                }
                            }
                        } else {
#pragma unroll
                            for (int c = 0; c < C; c++) {
                                const int j = (c + rot) & (C - 1);
                                if (2 * j + d <= n_m - 1)
                                    best[2 * c] = dmin(best[2 * c], __dadd_rn(U, rowS[2 * j + d]));
                                if (2 * j + 1 + d <= n_m - 1)
                                    best[2 * c + 1] = dmin(best[2 * c + 1], __dadd_rn(U, rowS[2 * j + 1 + d]));
                            }
                        }
                    }
                } else {
                    if (tr & (1 << 24)) {
                        const double2 x = *reinterpret_cast<const double2 *>(rowN + 2 * h);
                        best[0] = dmin(best[0], x.x);
                        best[1] = dmin(best[1], x.y);
                    }
                    const int m0 = 2 * h + d;
                    if (m0 <= n_m - 1) {
                        double y0, y1;
                        if ((d & 1) == 0) {
                            const double2 y = *reinterpret_cast<const double2 *>(rowS + m0);
                            y0 = y.x; y1 = y.y;
                        } else {
                            y0 = rowS[m0];
                            y1 = (m0 + 1 <= n_m - 1) ? rowS[m0 + 1] : MP_INF;
                        }
                        best[0] = dmin(best[0], __dadd_rn(U, y0));
                        if (m0 + 1 <= n_m - 1) best[1] = dmin(best[1], __dadd_rn(U, y1));
                    }
                }
            }
        }
        if (flags & 1) {   // tile complete: clamp (Q12) and store
            if (active) {
                const double tau = M.tau;
                double *o = M.out + (size_t)vv * M.rowlen + (size_t)pp_off * NMP;
                bool fin = false;
                if (ROW) {
#pragma unroll
                    for (int c = 0; c < C; c++) {
                        const int j = (c + rot) & (C - 1);
                        double2 r;
                        r.x = (2 * j < n_m && best[2 * c] <= tau) ? best[2 * c] : MP_INF;
                        r.y = (2 * j + 1 < n_m && best[2 * c + 1] <= tau) ? best[2 * c + 1] : MP_INF;
                        fin |= (r.x <= tau) | (r.y <= tau);
                        *reinterpret_cast<double2 *>(o + 2 * j) = r;
                    }
                } else {
                    double2 r;
                    r.x = (2 * h < n_m && best[0] <= tau) ? best[0] : MP_INF;
                    r.y = (2 * h + 1 < n_m && best[1] <= tau) ? best[1] : MP_INF;
                    fin = (r.x <= tau) | (r.y <= tau);
                    *reinterpret_cast<double2 *>(o + 2 * h) = r;
                }
                if (fin) atomicOr(M.flag + vv, 1u);
            }
#pragma unroll
            for (int i = 0; i < NB; i++) best[i] = MP_INF;
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * s);
        if (++s == nst) { s = 0; phase ^= 1; }
    }
}

// tile geometry of the persistent kernel (must match the consumer mapping above)
void persist_geom(int P, int n_v, int nmp, int *vb, int *np, int *n_ptiles, int *n_tiles) {
    const int rows = P - 1 > 0 ? P - 1 : 1;
    const int per_row = nmp <= 16 ? 1 : nmp / 2;      // threads per processor row
    int cap = kPCons / per_row;
    if (cap < 1) cap = 1;
    *np = rows < cap ? rows : cap;
    *n_ptiles = (rows + *np - 1) / *np;
    const int rowgroup = ((*np * per_row + 31) / 32) * 32;
    int v = kPCons / rowgroup;
    if (v < 1) v = 1;
    if (v > kMaxVb) v = kMaxVb;
    if (v > n_v) v = n_v;
    *vb = v;
    *n_tiles = ((n_v + *vb - 1) / *vb) * *n_ptiles;
}

// ring depth that fits in ~100 KB of dynamic shared memory (2 CTAs per SM)
int persist_nst(int stage_doubles) {
    int n = (96 * 1024) / (stage_doubles * 8);
    if (n > kNstMax) n = kNstMax;
    return n;   // the caller falls back to another step kernel if n < 2
}

void launch_step_persist(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp,
                         int stage_doubles, int nst, int grid, cudaStream_t s) {
    const int smem = nst * stage_doubles * 8;
    switch (nmp) {
#define MP_CASE(N)                                                                                      \
    case N:                                                                                             \
        cudaFuncSetAttribute(step_persist_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        step_persist_kernel<N><<<grid, kPCons + 32, smem, s>>>(jobs, tile_job, n_tiles, l, stage_doubles, nst); \
        break;
        MP_CASE(2) MP_CASE(4) MP_CASE(8) MP_CASE(16) MP_CASE(32) MP_CASE(64)
#undef MP_CASE
    }
}

int persist_blocks_per_sm(int nmp, int stage_doubles, int nst) {
    const int smem = nst * stage_doubles * 8;
    int n = 0;
    switch (nmp) {
#define MP_OCC(N)                                                                                       \
    case N:                                                                                             \
        cudaFuncSetAttribute(step_persist_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, step_persist_kernel<N>, kPCons + 32, smem);  \
        break;
        MP_OCC(2) MP_OCC(4) MP_OCC(8) MP_OCC(16) MP_OCC(32) MP_OCC(64)
#undef MP_OCC
    }
    return n < 1 ? 1 : n;
}

}  // namespace mp
