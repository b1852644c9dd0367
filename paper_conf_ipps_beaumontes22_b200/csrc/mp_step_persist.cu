// mp_step_persist.cu -- the wavefront min-plus step (a4-a5) as a persistent,
// warp-specialised, TMA-pipelined sm_100a kernel (the default step kernel).
//
// Same recursion as step_kernel (mp_kernels.cu), P:181-193 in decision form (Q1):
//   A[l][v][p][m] = clamp_tau( min over live k of
//        N: A[k-1][v'][p-1][m]            (normal GPU fits)
//        S: U(k,l) + A[k-1][v'][p][m+d]   (special GPU) ).
// The useful transitions (k, v) -> (v', nf, d) of layer l and the base row p = 0
// were computed beforehand by trans_kernel (a3, a4) into J.tlist / J.tcount.
//
// Structure:
//   * grid = resident CTAs (2 per SM).  A tile is vb delay rows x np processor rows of one job; every job of a launch
//     has the same P, hence the same tile geometry (passed as arguments).
//   * per-row sub-rings: delay row w of a tile owns a ring of nsg one-row slots in
//     shared memory, with its own full/empty mbarriers, consumed by its own warp
//     group.  Every slot carries exactly one useful source row segment, so the
//     bytes in flight per SM stay at the ring capacity whatever the liveness.
//   * warps 8.. are producers (n_prod, default 4); producer i feeds rings i, i+n_prod.  Per tile it reads, for each owned delay row, the list
//     of useful transitions prepared by trans_kernel (U(k,l), code, k in
//     ascending k) and issues, lane-parallel across rows and stages, one
//     cp.async.bulk per entry: the segment A[k-1][v'][p_lo-1 .. p_lo+np-1][*]
//     into the row's next slot, completing on the slot's mbarrier.  Tiles are
//     dealt to CTAs round-robin (tile_block = 1, measured best: candidates differ
//     in cost, interleaving balances them).
//   * warps 0-7 are consumers, one group per delay row.  ROW mode (NMP <= 16):
//     a thread owns one (v, p) row of NMP levels as NMP/2 16-byte chunks held in
//     a lane-rotated order (every quarter-warp's 16-byte shared loads hit 8
//     distinct bank groups; register indices stay compile-time).  PAIR mode
//     (NMP >= 32): a thread owns one (v, p, m-pair).  At the row's last stage
//     the group clamps to tau, stores, and flags the row finite/infinite.
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

constexpr int kSlotsMax = 64;        // one-row slots per CTA (all rings)
constexpr int kPCons = 256;          // consumer threads (8 warps)
constexpr int kProdMax = 4;          // producer warps (ring w is fed by producer w % n_prod)
constexpr int kMaxVb = 8;            // delay rows (= rings) per tile

struct SlotMeta {
    double *out;        // output row segment: A[l][v][p_lo][0]
    uint32_t *flag;     // row flag of (l, v)
    double tau;
    double U;           // U(k,l)
    int32_t tr;         // transition code
    int32_t np;         // processor rows of the tile (<= np_max)
    int16_t n_m, flags; // flags: 1 = last stage of the row, 2 = no data, 4 = terminate
    int32_t pad_;
};

template <int NMP>
__global__ void __launch_bounds__(kPCons + 32 * kProdMax, 2) step_persist_kernel(const Job *__restrict__ jobs,
                                                                      const int32_t *__restrict__ tile_job,
                                                                      int n_tiles, int l, int np_max, int vb,
                                                                      int nsg, unsigned long long *prof,
                                                                      int n_prod, int tile_block, size_t buf_off) {
    // prof (optional, MADPIPE_PROF=1): cycle counters [0] producer total, [1] tile setup,
    // [2] list building, [3] issue, [4] producer waits on empty, [5] consumer total,
    // [6] consumer waits on full, [7] tiles
    constexpr int C = NMP / 2;                       // 16-byte chunks per processor row
    constexpr bool ROW = NMP <= 16;
    constexpr int PER_ROW = ROW ? 1 : C;             // consumer threads per processor row
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ __align__(8) uint64_t full[kSlotsMax];
    __shared__ __align__(8) uint64_t empty[kSlotsMax];
    __shared__ SlotMeta meta[kSlotsMax];
    __shared__ Job pJs[kProdMax];                    // each producer's copy of its tile's job
    __shared__ int p_sl[kMaxVb], p_us[kMaxVb];       // per ring: next slot, its use count

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int rowgroup = ((np_max * PER_ROW + 31) / 32) * 32;   // threads per ring group
    const int wpg = rowgroup / 32;                               // warps per ring group
    const int seg_doubles = (np_max + 1) * NMP;                  // slot size
    const uint32_t full0 = smem_u32(&full[0]), empty0 = smem_u32(&empty[0]);
    const uint32_t ring_s = smem_u32(dsm);
    if (tid == 0) {
        for (int s = 0; s < vb * nsg; s++) {
            mbar_init(full0 + 8 * s, 1);
            mbar_init(empty0 + 8 * s, wpg);
        }
        for (int w = 0; w < kMaxVb; w++) { p_sl[w] = 0; p_us[w] = 0; }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const double *ring = reinterpret_cast<const double *>(dsm);

    if (warp >= kPCons / 32) {
        // ======================================================= producer warps
        const int pw = warp - kPCons / 32;           // producer index: rings pw, pw+kProd, ...
        Job &pJ = pJs[pw];
        const int my_rings = vb > pw ? (vb - pw + n_prod - 1) / n_prod : 0;
        const int lpr = my_rings > 0 ? 32 / my_rings : 32;   // lanes per owned ring
        const int m_round = min(nsg, lpr);           // stages per ring per issue round
        const int ir = lane / lpr, ij = lane - (lane / lpr) * lpr;
        const int iw = pw + ir * n_prod;             // the ring this lane serves
        long long t_p0 = clock64(), t_setup = 0, t_lists = 0, t_issue = 0, t_wempty = 0, n_tl = 0;
        int cur_jid = -1;
        // blocks of kTileBlock consecutive tiles, interleaved over the CTAs (balance +
        // job-descriptor reuse)
        for (int b0 = blockIdx.x * tile_block; b0 < n_tiles; b0 += gridDim.x * tile_block)
        for (int tile = b0; tile < min(n_tiles, b0 + tile_block); tile++) {
            if (my_rings == 0) break;
            long long ta = clock64();
            n_tl++;
            const int jid = tile_job[tile];
            if (jid != cur_jid) {   // cooperative copy of the job descriptor (one 8-byte word per lane)
                static_assert(sizeof(Job) % 8 == 0 && sizeof(Job) <= 32 * 8 * 2, "Job size");
                __syncwarp();
                const uint64_t *src = reinterpret_cast<const uint64_t *>(jobs + jid);
                uint64_t *dst = reinterpret_cast<uint64_t *>(&pJ);
                for (int w = lane; w < (int)(sizeof(Job) / 8); w += 32) dst[w] = __ldg(src + w);
                __syncwarp();
                cur_jid = jid;
            }
            const Job &J = pJ;
            if (l > J.L) continue;
            const int t = tile - J.tile0;
            const int vt = t / J.n_ptiles, pt = t - (t / J.n_ptiles) * J.n_ptiles;
            const int v0 = vt * J.vb;
            const int vcount = min(J.vb, J.n_v - v0);
            const int p_lo = 1 + pt * J.np;
            const int np = max(0, min(J.np, J.P - p_lo));
            if (np <= 0) continue;
            const size_t rowlen = (size_t)J.P * NMP;
            const size_t slab = (size_t)J.n_v * rowlen;
            const uint32_t seg_bytes = (uint32_t)(np + 1) * NMP * 8u;
            double *out = J.table + (size_t)l * slab;
            const bool my_ring = ir < my_rings && iw < vcount;
            // number of useful transitions of my ring's row (trans_kernel)
            // list buffer of layer l: buf_off entries (and buf_off / code_cap counts) in
            const int n_w = my_ring ? __ldg(J.tcount + buf_off / J.code_cap + v0 + iw) : 0;
            const TransEntry *list = J.tlist + buf_off + (size_t)(v0 + (my_ring ? iw : 0)) * J.code_cap;
            const int n_eff = my_ring ? (n_w > 0 ? n_w : 1) : 0;   // 1 = closing stage without data
            int max_n = n_eff;
            for (int o = 16; o > 0; o >>= 1) max_n = max(max_n, __shfl_xor_sync(0xffffffffu, max_n, o));
            if (prof) { const long long tb = clock64(); t_setup += tb - ta; ta = tb; }
            // ---- issue: lane (iw, ij) takes stages ij, ij+m, ... of ring iw
            for (int r0 = 0; r0 < max_n; r0 += m_round) {
                const int q = r0 + ij;
                if (my_ring && ij < m_round && q < n_eff) {
                    TransEntry e;
                    if (n_w > 0) e = list[q];
                    int s = p_sl[iw] + ij, use = p_us[iw];
                    if (s >= nsg) { s -= nsg; use++; }
                    const int slot = iw * nsg + s;
                    if (use > 0) {
                        const long long tw = prof ? clock64() : 0;
                        mbar_wait(empty0 + 8 * slot, (uint32_t)((use - 1) & 1));
                        if (prof && lane == 0) t_wempty += clock64() - tw;
                    }
                    SlotMeta &M = meta[slot];
                    M.out = out + (size_t)(v0 + iw) * rowlen + (size_t)p_lo * NMP;
                    M.flag = J.rowflag + (size_t)l * J.n_v + v0 + iw;
                    M.tau = J.tau;
                    M.np = np;
                    M.n_m = (int16_t)J.n_m;
                    if (n_w == 0) {
                        M.flags = 1 | 2;
                        M.tr = -1;
                        mbar_arrive(full0 + 8 * slot);
                    } else {
                        bulk_g2s(ring_s + 8u * (uint32_t)(slot * seg_doubles),
                                 J.table + (size_t)(e.k - 1) * slab + (size_t)(e.code & 0xFFFF) * rowlen +
                                     (size_t)(p_lo - 1) * NMP,
                                 seg_bytes, full0 + 8 * slot);
                        M.flags = (int16_t)(q == n_w - 1 ? 1 : 0);
                        M.tr = e.code;
                        M.U = e.U;
                        mbar_arrive_expect_tx(full0 + 8 * slot, seg_bytes);
                    }
                }
                __syncwarp();
                if (my_ring && ij == 0) {         // advance ring iw by the stages of this round
                    const int adv = max(0, min(m_round, n_eff - r0));
                    int s = p_sl[iw] + adv;
                    if (s >= nsg) { s -= nsg; p_us[iw]++; }
                    p_sl[iw] = s;
                }
                __syncwarp();
            }
            if (prof) { const long long tb = clock64(); t_issue += tb - ta; ta = tb; }
        }
        __syncwarp();
        if (prof && lane == 0 && pw == 0) {
            atomicAdd(prof + 0, (unsigned long long)(clock64() - t_p0));
            atomicAdd(prof + 1, (unsigned long long)t_setup);
            atomicAdd(prof + 2, (unsigned long long)t_lists);
            atomicAdd(prof + 3, (unsigned long long)t_issue);
            atomicAdd(prof + 4, (unsigned long long)t_wempty);
            atomicAdd(prof + 7, (unsigned long long)n_tl);
        }
        if (lane < my_rings) {   // terminate my rings
            const int w = pw + lane * n_prod;
            const int slot = w * nsg + p_sl[w];
            if (p_us[w] > 0) mbar_wait(empty0 + 8 * slot, (uint32_t)((p_us[w] - 1) & 1));
            meta[slot].flags = 4;
            mbar_arrive(full0 + 8 * slot);
        }
        return;
    }

    // =========================================================== consumer warps
    const int grp = warp / wpg;                      // my ring
    if (grp >= vb) return;                           // idle warps (vb * wpg < 8)
    const int q = tid - grp * rowgroup;
    int pp_off, h = 0, rot = 0;
    if (ROW) {
        pp_off = q;
        constexpr int G8 = C >= 8 ? 1 : 8 / C;       // lanes sharing a 128-byte window
        constexpr int RM = C >= 8 ? 8 : C;
        rot = (pp_off / G8) % RM;
    } else {
        pp_off = q / C;
        h = q - pp_off * C;
    }
    constexpr int NB = ROW ? NMP : 2;                // accumulators per thread
    double best[NB];
#pragma unroll
    for (int i = 0; i < NB; i++) best[i] = MP_INF;
    int s = 0, phase = 0;
    const long long t_c0 = clock64();
    long long t_wfull = 0;
    for (;;) {
        const int slot = grp * nsg + s;
        const long long tw = prof ? clock64() : 0;
        mbar_wait(full0 + 8 * slot, (uint32_t)phase);
        if (prof) t_wfull += clock64() - tw;
        const SlotMeta &M = meta[slot];
        const int flags = M.flags;
        if (flags & 4) {
            if (prof && lane == 0 && warp == 0) {
                atomicAdd(prof + 5, (unsigned long long)(clock64() - t_c0));
                atomicAdd(prof + 6, (unsigned long long)t_wfull);
            }
            break;
        }
        const int np = M.np, n_m = M.n_m;
        const bool active = pp_off < np;
        if (!(flags & 2) && active) {
            const int32_t tr = M.tr;
            const double *rowN = ring + (size_t)slot * seg_doubles + pp_off * NMP;   // processor p-1
            const double *rowS = rowN + NMP;                                          // processor p
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
        if (flags & 1) {   // row complete: clamp (Q12), store, flag
            bool fin = false;
            if (active) {
                const double tau = M.tau;
                double *o = M.out + (size_t)pp_off * NMP;
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
            }
            if (__ballot_sync(0xffffffffu, fin) && lane == 0) atomicOr(M.flag, 1u);
#pragma unroll
            for (int i = 0; i < NB; i++) best[i] = MP_INF;
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * slot);
        if (++s == nsg) { s = 0; phase ^= 1; }
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

// slots per ring: as many one-row slots as fit in ~96 KB, split over the vb rings
int persist_nsg(int np, int vb, int nmp) {
    const int seg = (np + 1) * nmp * 8;
    int slots = (96 * 1024) / seg;
    if (slots > kSlotsMax) slots = kSlotsMax;
    return slots / vb;   // the caller falls back to another step kernel if < 2
}

void launch_step_persist(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp, int np,
                         int vb, int nsg, int grid, unsigned long long *prof, int n_prod, int tile_block,
                         size_t buf_off, cudaStream_t s) {
    const int smem = vb * nsg * (np + 1) * nmp * 8;
    switch (nmp) {
#define MP_CASE(N)                                                                                      \
    case N:                                                                                             \
        cudaFuncSetAttribute(step_persist_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        step_persist_kernel<N><<<grid, kPCons + 32 * n_prod, smem, s>>>(jobs, tile_job, n_tiles, l, np, vb, nsg, prof, n_prod, tile_block, buf_off); \
        break;
        MP_CASE(2) MP_CASE(4) MP_CASE(8) MP_CASE(16) MP_CASE(32) MP_CASE(64)
#undef MP_CASE
    }
}

int persist_blocks_per_sm(int nmp, int np, int vb, int nsg, int n_prod) {
    const int smem = vb * nsg * (np + 1) * nmp * 8;
    int n = 0;
    switch (nmp) {
#define MP_OCC(N)                                                                                       \
    case N:                                                                                             \
        cudaFuncSetAttribute(step_persist_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, step_persist_kernel<N>, kPCons + 32 * n_prod, smem);  \
        break;
        MP_OCC(2) MP_OCC(4) MP_OCC(8) MP_OCC(16) MP_OCC(32) MP_OCC(64)
#undef MP_OCC
    }
    return n < 1 ? 1 : n;
}

}  // namespace mp
