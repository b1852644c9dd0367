// mp_step_persist.cu -- the wavefront min-plus step (a3-a5) as a persistent,
// warp-specialised, TMA-pipelined sm_100a kernel.
//
// Same recursion as step_kernel (mp_kernels.cu), P:181-193 in decision form (Q1):
//   A[l][v][p][m] = clamp_tau( min over live k of
//        N: A[k-1][v'][p-1][m]            (normal GPU fits)
//        S: U(k,l) + A[k-1][v'][p][m+d]   (special GPU) ).
//
// Structure:
//   * grid = resident CTAs (a few per SM); CTA c takes tiles c, c+G, c+2G, ...
//     A tile is vb delay rows x np processor rows of one job (same geometry as
//     the non-persistent TMA kernel).
//   * warp 8 is the producer.  For each tile it computes the live transitions
//     (k, v) of the window with all 32 lanes (a3), writes the base row p = 0
//     (a4), and for every k with a live row streams the source row segments
//     A[k-1][v'][p_lo-1 .. p_lo+np-1][*] into an NST-stage shared-memory ring
//     with cp.async.bulk, completing on the stage's mbarrier.  Per-stage
//     metadata (the tile's output row, tau, the transition codes, U(k,l))
//     travels in a small shared-memory array next to the ring.
//   * warps 0-7 are consumers: each thread owns a (p, m-pair) of one delay row,
//     so the shift d is warp-uniform.  N is one 16-byte shared load, S one
//     16-byte (d even) or two 8-byte (d odd) loads + DADD; two min's per level.
//     At the tile's last stage they clamp to tau and store.
//   * the ring never drains between tiles, so each SM keeps NST x CTAs row
//     segments in flight (Little's law for HBM latency).
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
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

}  // namespace

constexpr int kPNst = 8;             // ring stages
constexpr int kG = 4;                // source k-rows (x delay rows) per stage
constexpr int kPCons = 256;          // consumer threads
constexpr int kMaxVb = 8;            // delay rows per tile (host geometry caps at this)
constexpr int kMaxGroups = 512;      // live k per tile (window <= L <= 512 layers)

// per-stage metadata written by the producer, read by the consumers
struct StageMeta {
    double *out;              // output row of delay v0 (row v0+vv at out + vv*rowlen)
    double tau;
    double U[kG];             // U(k,l) of each k of the stage
    int32_t tr[kG][kMaxVb];   // transition code per (k, delay row) (<0: not live)
    int32_t rowlen;           // P*NMP
    int16_t np, vcount, n_m, flags;   // flags: 1 = last stage of the tile, 2 = no data, 4 = terminate
    int16_t ng, pad_[3];      // k-rows in this stage
};

template <int NMP>
__global__ void __launch_bounds__(kPCons + 32, 2) step_persist_kernel(const Job *__restrict__ jobs,
                                                                      const int32_t *__restrict__ tile_job,
                                                                      int n_tiles, int l, int stage_doubles) {
    constexpr int HP = NMP / 2;
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ __align__(8) uint64_t full[kPNst];
    __shared__ __align__(8) uint64_t empty[kPNst];
    __shared__ StageMeta meta[kPNst];
    __shared__ Job pJ;              // producer's copy of the current tile's job
    __shared__ int32_t p_tr[kMaxGroups * kMaxVb];   // live codes of the tile's groups
    __shared__ int32_t p_grp[kMaxGroups];           // k of each group

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    if (tid == 0) {
        for (int s = 0; s < kPNst; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kPCons / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    double *ring = reinterpret_cast<double *>(dsm);

    if (warp == kPCons / 32) {
        // =================================================== producer warp
        // Phase A (all lanes): live transitions of the tile's window -> p_grp
        // (compacted k with at least one live delay row) and p_tr (codes).
        // Phase B (lane-parallel): lane i issues stage gi+i for group i.
        int gi = 0;
        for (int tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
            const int jid = tile_job[tile];
            __syncwarp();
            if (lane == 0) pJ = jobs[jid];
            __syncwarp();
            const Job &J = pJ;
            if (l > J.L) continue;
            const int t = tile - J.tile0;
            const int vt = t / J.n_ptiles, pt = t % J.n_ptiles;
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
            if (pt == 0 && lane < vcount) {       // base row p = 0 (Q10)
                const int v = v0 + lane;
                const double U1l = __dsub_rn(Ul, J.Up[0]);
                int64_t d;
                (void)transition(J, 1, l, v, U1l, &d);
                double *o = out + (size_t)v * rowlen;
#pragma unroll
                for (int m = 0; m < NMP; m++)
                    o[m] = (m < n_m && U1l <= tau && (int64_t)m + d <= (int64_t)(n_m - 1)) ? U1l : MP_INF;
            }
            if (np <= 0) continue;
            // ---- phase A: read the precomputed codes of the window (trans_kernel)
            const int kmin = *J.kmin_l;
            const int wl = l + 1 - kmin;
            const int per = 32 / vcount;                 // k per pass (vcount <= 8)
            const int kk = lane / vcount, v2 = lane - kk * vcount;
            const unsigned grp_mask = ((1u << vcount) - 1u) << (kk * vcount);
            const int32_t *codes = J.codes + (size_t)(v0 + v2) * J.code_cap;
            for (int kb = kmin; kb <= l;) {
                // collect up to kMaxGroups live groups
                int ngrp = 0;
                for (; kb <= l && ngrp + per <= kMaxGroups; kb += per) {
                    const int k = kb + kk;
                    const bool valid = kk < per && k <= l;
                    const int32_t tr = valid ? codes[k - kmin] : -1;
                    const unsigned live = __ballot_sync(0xffffffffu, tr >= 0);
                    const bool leader = valid && (v2 == 0) && (live & grp_mask);
                    const unsigned leaders = __ballot_sync(0xffffffffu, leader);
                    const int rank = ngrp + __popc(leaders & ((1u << lane) - 1u));
                    const int myrank = __shfl_sync(0xffffffffu, rank, valid ? kk * vcount : 0);
                    if (valid && (live & grp_mask)) {
                        p_tr[myrank * kMaxVb + v2] = tr;
                        if (v2 == 0) p_grp[myrank] = k;
                    }
                    ngrp += __popc(leaders);
                }
                const bool done = kb > l;
                __syncwarp();
                // phase B: stages of up to kG live groups; the tile's last stage carries
                // flag 1 (an empty closing stage if the final chunk has no live group).
                // Rounds of at most kPNst stages: the slots of one round are distinct, so
                // each lane's parity wait refers to the previous use of its own slot (a
                // lane must never wait two phases ahead: mbarrier parity would alias).
                const int nst = ngrp > 0 ? (ngrp + kG - 1) / kG : (done ? 1 : 0);
                for (int g0 = 0; g0 < nst; g0 += kPNst) {
                    const int g = g0 + lane;
                    if (lane < kPNst && g < nst) {
                        const int gg = gi + g;
                        const int s = gg % kPNst;
                        if (gg >= kPNst) mbar_wait(&empty[s], (uint32_t)((gg / kPNst - 1) & 1));
                        StageMeta &M = meta[s];
                        M.out = out + (size_t)v0 * rowlen + (size_t)p_lo * NMP;
                        M.tau = tau;
                        M.rowlen = (int32_t)rowlen;
                        M.np = (int16_t)np; M.vcount = (int16_t)vcount; M.n_m = (int16_t)n_m;
                        M.flags = (int16_t)((done && g == nst - 1 ? 1 : 0) | (ngrp == 0 ? 2 : 0));
                        if (ngrp == 0) {
                            M.ng = 0;
                            mbar_arrive(&full[s]);
                        } else {
                            const int q0 = g * kG;
                            const int ng = min(kG, ngrp - q0);
                            M.ng = (int16_t)ng;
                            uint32_t bytes = 0;
                            for (int q = 0; q < ng; q++) {
                                const int k = p_grp[q0 + q];
                                M.U[q] = __dsub_rn(Ul, J.Up[k - 1]);
                                const double *src_slab =
                                    J.table + (size_t)(k - 1) * slab + (size_t)(p_lo - 1) * NMP;
                                for (int w = 0; w < kMaxVb; w++) {
                                    const int32_t trw = w < vcount ? p_tr[(q0 + q) * kMaxVb + w] : -1;
                                    M.tr[q][w] = trw;
                                    if (trw < 0) continue;
                                    bytes += seg_bytes;
                                    bulk_g2s(ring + (size_t)s * stage_doubles + (size_t)(q * vcount + w) * seg_doubles,
                                             src_slab + (size_t)(trw & 0xFFFF) * rowlen, seg_bytes, &full[s]);
                                }
                            }
                            mbar_arrive_expect_tx(&full[s], bytes);
                        }
                    }
                    __syncwarp();
                }
                gi += nst;
                if (done) break;
            }
            (void)wl;
            if (kmin > l) {   // empty window: close the tile
                if (lane == 0) {
                    const int s = gi % kPNst;
                    if (gi >= kPNst) mbar_wait(&empty[s], (uint32_t)((gi / kPNst - 1) & 1));
                    StageMeta &M = meta[s];
                    M.out = out + (size_t)v0 * rowlen + (size_t)p_lo * NMP;
                    M.tau = tau;
                    M.rowlen = (int32_t)rowlen;
                    M.np = (int16_t)np; M.vcount = (int16_t)vcount; M.n_m = (int16_t)n_m;
                    M.flags = 1 | 2;
                    M.ng = 0;
                    mbar_arrive(&full[s]);
                }
                gi += 1;
            }
        }
        __syncwarp();
        if (lane == 0) {
            const int s = gi % kPNst;
            if (gi >= kPNst) mbar_wait(&empty[s], (uint32_t)((gi / kPNst - 1) & 1));
            meta[s].flags = 4;
            mbar_arrive(&full[s]);
        }
        return;
    }

    // ======================================================= consumer warps
    double best0 = MP_INF, best1 = MP_INF;
    int cur_np = -1, cur_vc = -1, vv = 0, pp_off = 0, h = 0;
    bool active = false;
    for (int gi = 0;; gi++) {
        const int s = gi % kPNst;
        mbar_wait(&full[s], (uint32_t)((gi / kPNst) & 1));
        const StageMeta &M = meta[s];
        const int flags = M.flags;
        if (flags & 4) break;
        const int np = M.np, vcount = M.vcount, n_m = M.n_m;
        if (np != cur_np || vcount != cur_vc) {
            const int rowgroup = ((np * HP + 31) / 32) * 32;
            vv = tid / rowgroup;
            const int q = tid - vv * rowgroup;
            pp_off = q / HP;
            h = q - pp_off * HP;
            active = vv < vcount && pp_off < np;
            cur_np = np; cur_vc = vcount;
        }
        if (!(flags & 2) && active) {
            const int ng = M.ng;
            for (int q = 0; q < ng; q++) {
                const int32_t tr = M.tr[q][vv];
                if (tr < 0) continue;
                const double *seg = ring + (size_t)s * stage_doubles + (size_t)(q * vcount + vv) * (np + 1) * NMP;
                if (tr & (1 << 24)) {
                    const double2 x = *reinterpret_cast<const double2 *>(seg + pp_off * NMP + 2 * h);
                    best0 = x.x < best0 ? x.x : best0;
                    best1 = x.y < best1 ? x.y : best1;
                }
                const int d = (tr >> 16) & 0xFF;
                const int m0 = 2 * h + d;
                if (m0 <= n_m - 1) {
                    const double U = M.U[q];
                    const double *r = seg + (pp_off + 1) * NMP;
                    double y0, y1;
                    if ((d & 1) == 0) {
                        const double2 y = *reinterpret_cast<const double2 *>(r + m0);
                        y0 = y.x; y1 = y.y;
                    } else {
                        y0 = r[m0];
                        y1 = (m0 + 1 <= n_m - 1) ? r[m0 + 1] : MP_INF;
                    }
                    const double c0 = __dadd_rn(U, y0);
                    best0 = c0 < best0 ? c0 : best0;
                    if (m0 + 1 <= n_m - 1) {
                        const double c1 = __dadd_rn(U, y1);
                        best1 = c1 < best1 ? c1 : best1;
                    }
                }
            }
        }
        if (flags & 1) {   // tile complete: clamp (Q12) and store
            if (active) {
                double2 r;
                r.x = (2 * h < n_m && best0 <= M.tau) ? best0 : MP_INF;
                r.y = (2 * h + 1 < n_m && best1 <= M.tau) ? best1 : MP_INF;
                *reinterpret_cast<double2 *>(M.out + (size_t)vv * M.rowlen + (size_t)pp_off * NMP + 2 * h) = r;
            }
            best0 = MP_INF;
            best1 = MP_INF;
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[s]);
    }
}

int persist_group_rows() { return kG; }

int persist_smem_bytes(int stage_doubles) { return kPNst * stage_doubles * 8; }

void launch_step_persist(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp,
                         int stage_doubles, int grid, cudaStream_t s) {
    const int smem = persist_smem_bytes(stage_doubles);
    switch (nmp) {
#define MP_CASE(N)                                                                                      \
    case N:                                                                                             \
        cudaFuncSetAttribute(step_persist_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        step_persist_kernel<N><<<grid, kPCons + 32, smem, s>>>(jobs, tile_job, n_tiles, l, stage_doubles); \
        break;
        MP_CASE(2) MP_CASE(4) MP_CASE(8) MP_CASE(16) MP_CASE(32) MP_CASE(64)
#undef MP_CASE
    }
}

int persist_blocks_per_sm(int nmp, int stage_doubles) {
    const int smem = persist_smem_bytes(stage_doubles);
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
