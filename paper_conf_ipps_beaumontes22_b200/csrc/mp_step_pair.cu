// mp_step_pair.cu -- the wavefront min-plus step (a3-a5) blocked over TWO layers:
// one pass computes layer l and layer l+1 (all options k <= l), so a source row
// A[k-1][v'] that both layers read is brought on chip once.
//
// Same recursion as step_persist_kernel, P:181-193 in decision form (Q1):
//   A[l][v][p][m] = clamp_tau( min over live k of
//        N: A[k-1][v'][p-1][m]            (normal GPU fits)
//        S: U(k,l) + A[k-1][v'][p][m+d]   (special GPU) ).
// Why two layers share sources: layer l+1's delay row w enters stage k..l+1 with
// V_w + U(k,l) + u_{l+1}, layer l's row v with V_v + U(k,l); for w = v - delta,
// delta = round(u_{l+1} / dV), both land on (nearly always) the same next level
// v' = ceil(((V (+) U) (+) C(k-1)) / dV) of P:179.  Measured at GPT: a 2x8-row
// tile loads ~1.9x fewer source rows than the two layers separately.
//
// Layer l+1's option k = l+1 reads slab l, which this pass is writing, so the
// pass stores layer l+1 without it (clamped; clamp and min commute, Q12) and
// pair_fixup_kernel applies it afterwards: one extra read+write of slab l+1.
// min is exact and order-free, so every value equals the oracle's bit for bit.
//
// Kernels:
//   pair_trans_kernel : one warp per (job, v-tile): base rows p = 0 of both
//                       layers, row-flag reset, and the tile's merged list of useful
//                       source rows (k, v') with a row mask and per-row (d, nf).
//   pair_step_kernel  : persistent, 1 CTA per SM: one producer warp streams each
//                       list entry's source segment A[k-1][v'][p_lo-1 .. p_lo+np-1][*]
//                       into a shared ring with cp.async.bulk (TMA bulk copy);
//                       16 consumer warps, one per output row of the tile, each
//                       thread owning processor rows p_lo+lane and p_lo+32+lane.
//   pair_fixup_kernel : one warp per (job, v) of layer l+1: option k = l+1.
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

constexpr int kPairVB = 8;                       // delay rows per layer in a tile
constexpr int kPairRows = 2 * kPairVB;           // output rows (= consumer warps) per tile
constexpr int kPairE = 2;                        // extra v-tiles: layer l+1 rows are shifted by <= kPairE*kPairVB
constexpr int kPairNp = 64;                      // processor rows per tile (2 per consumer thread)
constexpr int kPairSlotsMax = 64;
constexpr int kPairThreads = 32 * (kPairRows + 1);

// One source row of a tile's merged list (pair_trans_kernel -> pair_step_kernel).
struct PairEntry {
    uint16_t k;        // option k: the source is slab k-1
    uint16_t vp;       // next delay level v' (source row)
    uint16_t mask;     // output rows of the tile that read it (bit r: r < 8 layer l, else l+1)
    uint16_t pad;
    uint8_t code[kPairRows];   // per row: d (bits 0-6, clamped to 127) | nf << 7
};
static_assert(sizeof(PairEntry) == 24, "PairEntry size");

// delta of layer pair (l, l+1): layer l+1's rows of v-tile t are v0 - delta ..
// (any delta is correct; this one maximises shared source rows).  Clamped so that
// kPairE extra tiles always cover layer l+1.
__device__ __forceinline__ int pair_shift(const Job &J, int l) {
    if (l + 1 > J.L) return 0;
    const double q = rint(__ddiv_rn(__dsub_rn(J.Up[l + 1], J.Up[l]), J.dV));
    if (!(q > 0.0)) return 0;
    return q > (double)(kPairE * kPairVB) ? kPairE * kPairVB : (int)q;
}

__device__ __forceinline__ int pair_vtiles(int n_v) { return (n_v + kPairVB - 1) / kPairVB + kPairE; }

// ---------------------------------------------------------------------------
// a3 + a4 for the layer pair (l, l+1).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(128) pair_trans_kernel(const Job *jobs, int l, int nmp, size_t buf_off,
                                                         size_t cnt_off) {
    __shared__ Job sJ;
    if (threadIdx.x < sizeof(Job) / 8)
        reinterpret_cast<uint64_t *>(&sJ)[threadIdx.x] =
            __ldg(reinterpret_cast<const uint64_t *>(jobs + blockIdx.y) + threadIdx.x);
    __syncthreads();
    const Job &J = sJ;
    if (l > J.L) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int vt = blockIdx.x * 4 + warp;
    if (vt >= pair_vtiles(J.n_v)) return;
    const bool hasB = l + 1 <= J.L;
    const int delta = pair_shift(J, l);
    const int r = lane & 15, h = lane >> 4;      // row r of the tile; half h takes k = kb + h
    const bool isB = r >= kPairVB;
    const int lr = isB ? l + 1 : l;              // the row's layer
    const int v = isB ? vt * kPairVB - delta + (r - kPairVB) : vt * kPairVB + r;
    const bool row_ok = (!isB || hasB) && v >= 0 && v < J.n_v;
    const size_t rowlen = (size_t)J.P * nmp;
    const size_t slab = (size_t)J.n_v * rowlen;
    const double Ulr = J.Up[lr];
    // base row p = 0 (reading Q10) and the row flag, OR-ed later for p >= 1
    if (row_ok && h == 0) {
        const double U1l = __dsub_rn(Ulr, J.Up[0]);
        int64_t d;
        (void)transition(J, 1, lr, v, U1l, &d);
        const bool ok = U1l <= J.tau && d <= (int64_t)(J.n_m - 1);
        double *o = J.table + (size_t)lr * slab + (size_t)v * rowlen;
        for (int m = 0; m < nmp; m++)
            o[m] = (m < J.n_m && U1l <= J.tau && (int64_t)m + d <= (int64_t)(J.n_m - 1)) ? U1l : MP_INF;
        J.rowflag[(size_t)lr * J.n_v + v] = ok ? 1u : 0u;
    }
    const int kA = J.kwin[l];                    // window starts max(kmin_tau, kmin_W)
    const int kw = isB ? (hasB ? J.kwin[l + 1] : l + 1) : kA;
    unsigned live = 0, useful = 0;
    int n = 0;
    PairEntry *list = reinterpret_cast<PairEntry *>(J.tlist) + buf_off + (size_t)vt * J.code_cap;
    for (int kb = kA; kb <= l; kb += 2) {        // k <= l: sources in slabs <= l-1 (final)
        const int k = kb + h;
        int key = -1 - lane;                     // unique unless the row reads a source
        uint32_t code = 0;
        if (row_ok && k <= l && k >= kw) {
            int64_t d;
            const int32_t tr = transition(J, k, lr, v, __dsub_rn(Ulr, J.Up[k - 1]), &d);
            if (tr >= 0) {
                live++;
                const int vn = tr & 0xFFFF;
                // a source row that is +inf everywhere contributes +inf (exact skip)
                if (J.rowflag[(size_t)(k - 1) * J.n_v + vn] != 0u) {
                    useful++;
                    key = (k << 16) | vn;
                    code = (uint32_t)(d > 127 ? 127 : d) | ((tr >> 24) & 1u) << 7;
                }
            }
        }
        const unsigned grp = __match_any_sync(0xffffffffu, key);
        const int leader = __ffs(grp) - 1;
        const bool lead = key >= 0 && leader == lane;
        const unsigned lb = __ballot_sync(0xffffffffu, lead);
        int idx = n + __popc(lb & ((1u << lane) - 1u));
        idx = __shfl_sync(0xffffffffu, idx, leader);
        if (lead) {
            const uint64_t head = (uint64_t)(uint32_t)k | (uint64_t)(uint32_t)(key & 0xFFFF) << 16 |
                                  (uint64_t)((grp >> (16 * h)) & 0xFFFFu) << 32;
            *reinterpret_cast<uint64_t *>(list + idx) = head;
        }
        if (key >= 0) list[idx].code[r] = (uint8_t)code;
        n += __popc(lb);
    }
    if (lane == 0) J.tcount[cnt_off + vt] = n;
    for (int o = 16; o > 0; o >>= 1) {
        live += __shfl_xor_sync(0xffffffffu, live, o);
        useful += __shfl_xor_sync(0xffffffffu, useful, o);
    }
    if (lane == 0 && live && J.P > 1) {
        const unsigned long long per = (unsigned long long)(J.P - 1) * (unsigned long long)J.n_m;
        atomicAdd(J.eff, (unsigned long long)live * per);
        if (useful) atomicAdd(J.useful, (unsigned long long)useful * per);
    }
    if (lane == 0 && n && J.segs) atomicAdd(J.segs, (unsigned long long)n);
}

// ---------------------------------------------------------------------------
// a5 for the layer pair: the persistent two-layer step kernel.
// ---------------------------------------------------------------------------
struct PairMeta {
    uint32_t mask;          // rows reading this slot's source segment
    int16_t flags;          // 0 = data, 1 = tile end (store the rows), 4 = terminate
    int16_t np;             // processor rows of the tile
    union {
        struct { double U0, U1; uint8_t code[kPairRows]; } e;       // data: U(k,l), U(k,l+1), codes
        struct { double tau; double *outA; uint32_t *flA; int32_t v0A, v0B; } t;  // tile end
    };
    int64_t slab;           // doubles per slab
    int32_t rowlen, n_v;
    int32_t hasB, n_m;
};
static_assert(sizeof(PairMeta) == 64, "PairMeta size");

// relax one processor row of NMP levels held in lane-rotated chunk order
// (same arithmetic and layout as step_persist_kernel's ROW mode)
template <int NMP>
__device__ __forceinline__ void pair_relax(double (&best)[NMP], const double *rowN, int rot, int d, bool nf,
                                           double U, int n_m) {
    constexpr int C = NMP / 2;
    const double *rowS = rowN + NMP;
    if (nf) {                                                    // N
#pragma unroll
        for (int c = 0; c < C; c++) {
            const int j = (c + rot) & (C - 1);
            const double2 x = *reinterpret_cast<const double2 *>(rowN + 2 * j);
            best[2 * c] = dmin(best[2 * c], x.x);
            best[2 * c + 1] = dmin(best[2 * c + 1], x.y);
        }
    }
    if (d <= n_m - 1) {                                          // S
        if ((d & 1) == 0) {
            const int e = d >> 1;
#pragma unroll
            for (int c = 0; c < C; c++) {
                const int j = (c + rot) & (C - 1);
                if (2 * j + d <= n_m - 1) {
                    const double2 y = *reinterpret_cast<const double2 *>(rowS + 2 * (j + e));
                    best[2 * c] = dmin(best[2 * c], __dadd_rn(U, y.x));
                    if (2 * j + 1 + d <= n_m - 1) best[2 * c + 1] = dmin(best[2 * c + 1], __dadd_rn(U, y.y));
                }
            }
        } else {
#pragma unroll
            for (int c = 0; c < C; c++) {
                const int j = (c + rot) & (C - 1);
                if (2 * j + d <= n_m - 1) best[2 * c] = dmin(best[2 * c], __dadd_rn(U, rowS[2 * j + d]));
                if (2 * j + 1 + d <= n_m - 1)
                    best[2 * c + 1] = dmin(best[2 * c + 1], __dadd_rn(U, rowS[2 * j + 1 + d]));
            }
        }
    }
}

// clamp (Q12) and store one processor row; returns whether a value is finite
template <int NMP>
__device__ __forceinline__ bool pair_store(double (&best)[NMP], double *o, int rot, double tau, int n_m) {
    constexpr int C = NMP / 2;
    bool fin = false;
#pragma unroll
    for (int c = 0; c < C; c++) {
        const int j = (c + rot) & (C - 1);
        double2 r;
        r.x = (2 * j < n_m && best[2 * c] <= tau) ? best[2 * c] : MP_INF;
        r.y = (2 * j + 1 < n_m && best[2 * c + 1] <= tau) ? best[2 * c + 1] : MP_INF;
        fin |= (r.x <= tau) | (r.y <= tau);
        *reinterpret_cast<double2 *>(o + 2 * j) = r;
    }
#pragma unroll
    for (int i = 0; i < NMP; i++) best[i] = MP_INF;
    return fin;
}

template <int NMP>
__global__ void __launch_bounds__(kPairThreads, 1) pair_step_kernel(const Job *__restrict__ jobs,
                                                                    const int32_t *__restrict__ tile_job,
                                                                    int n_tiles, int l, int np_max, int nsl,
                                                                    int round, size_t buf_off, size_t cnt_off) {
    // Slots are shared by the rows that read them: the producer pushes each slot
    // (with the parity of its full-barrier phase) into the queue of every row in
    // its mask; a row warp visits only its own slots; the last reader (reference
    // count) releases the slot's empty barrier.  Tile ends and the final
    // termination are slots without data pushed to all 16 rows.
    constexpr int C = NMP / 2;
    constexpr int QN = 64;                                 // queue entries per row (>= slots)
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ __align__(8) uint64_t full[kPairSlotsMax];
    __shared__ __align__(8) uint64_t empty[kPairSlotsMax];
    __shared__ __align__(16) PairMeta meta[kPairSlotsMax];
    __shared__ __align__(16) Job pJ;
    __shared__ uint8_t rq[kPairRows][QN];                  // per-row queues: slot | phase parity << 7
    __shared__ int rtail[kPairRows];                       // entries pushed per row (producer)
    __shared__ int sref[kPairSlotsMax];                    // readers left per slot

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int seg_doubles = (np_max + 1) * NMP;
    const uint32_t full0 = smem_u32(&full[0]), empty0 = smem_u32(&empty[0]);
    const uint32_t ring_s = smem_u32(dsm);
    if (tid == 0) {
        for (int s = 0; s < nsl; s++) {
            mbar_init(full0 + 8 * s, 1);
            mbar_init(empty0 + 8 * s, 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tid < kPairRows) rtail[tid] = 0;
    __syncthreads();
    const double *ring = reinterpret_cast<const double *>(dsm);
    volatile int *vtail = rtail;

    if (warp == kPairRows) {
        // =========================================================== producer warp
        int sl = 0, wraps = 0, cur = -1;
        int my_tail = 0;                                   // lane r < 16: entries pushed to row r
        const unsigned lt = (1u << lane) - 1u;
        auto push = [&](bool act, uint32_t mask, uint32_t ent) {
            // append ent to the queue of every row in mask, in lane order
#pragma unroll
            for (int rr = 0; rr < kPairRows; rr++) {
                const bool mine = act && ((mask >> rr) & 1u);
                const unsigned bal = __ballot_sync(0xffffffffu, mine);
                const int base = __shfl_sync(0xffffffffu, my_tail, rr);
                if (mine) rq[rr][(base + __popc(bal & lt)) & (QN - 1)] = (uint8_t)ent;
                if (lane == rr) my_tail += __popc(bal);
            }
            __syncwarp();
            __threadfence_block();
            if (lane < kPairRows) vtail[lane] = my_tail;
        };
        for (int tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
            const int jid = tile_job[tile];
            if (jid != cur) {
                __syncwarp();
                const uint64_t *src = reinterpret_cast<const uint64_t *>(jobs + jid);
                uint64_t *dst = reinterpret_cast<uint64_t *>(&pJ);
                for (int w = lane; w < (int)(sizeof(Job) / 8); w += 32) dst[w] = __ldg(src + w);
                __syncwarp();
                cur = jid;
            }
            const Job &J = pJ;
            if (l > J.L) continue;
            const int t = tile - J.tile0;
            const int vt = t / J.n_ptiles, pt = t - (t / J.n_ptiles) * J.n_ptiles;
            const int p_lo = 1 + pt * np_max;
            const int np = min(np_max, J.P - p_lo);
            if (np <= 0) continue;
            const bool hasB = l + 1 <= J.L;
            const int delta = pair_shift(J, l);
            const int64_t rowlen = (int64_t)J.P * NMP;
            const int64_t slab = (int64_t)J.n_v * rowlen;
            const uint32_t seg_bytes = (uint32_t)(np + 1) * NMP * 8u;
            const int n = __ldg(J.tcount + cnt_off + vt);
            const PairEntry *list = reinterpret_cast<const PairEntry *>(J.tlist) + buf_off + (size_t)vt * J.code_cap;
            const double Ul = J.Up[l], Ul1 = hasB ? J.Up[l + 1] : 0.0;
            const int stages = n + 1;                      // entries, then the tile-end marker
            for (int r0 = 0; r0 < stages; r0 += round) {
                const int q = r0 + lane;
                const bool act = lane < round && q < stages;
                uint32_t mask = 0, ent = 0;
                if (act) {
                    int s = sl + lane, use = wraps;
                    if (s >= nsl) { s -= nsl; use++; }
                    if (use > 0) mbar_wait(empty0 + 8 * s, (uint32_t)((use - 1) & 1));
                    ent = (uint32_t)s | (uint32_t)(use & 1) << 7;
                    PairMeta &M = meta[s];
                    M.np = (int16_t)np;
                    M.n_m = J.n_m;
                    if (q < n) {
                        const uint64_t *ep = reinterpret_cast<const uint64_t *>(list + q);
                        const uint64_t head = __ldg(ep);
                        const int k = (int)(head & 0xFFFFu), vp = (int)((head >> 16) & 0xFFFFu);
                        bulk_g2s(ring_s + 8u * (uint32_t)(s * seg_doubles),
                                 J.table + (int64_t)(k - 1) * slab + (int64_t)vp * rowlen + (int64_t)(p_lo - 1) * NMP,
                                 seg_bytes, full0 + 8 * s);
                        mask = (uint32_t)(head >> 32) & 0xFFFFu;
                        M.mask = mask;
                        M.flags = 0;
                        const double Uk = J.Up[k - 1];
                        M.e.U0 = __dsub_rn(Ul, Uk);
                        M.e.U1 = hasB ? __dsub_rn(Ul1, Uk) : 0.0;
                        reinterpret_cast<uint64_t *>(M.e.code)[0] = __ldg(ep + 1);
                        reinterpret_cast<uint64_t *>(M.e.code)[1] = __ldg(ep + 2);
                        sref[s] = __popc(mask);
                        mbar_arrive_expect_tx(full0 + 8 * s, seg_bytes);
                    } else {
                        mask = (1u << kPairRows) - 1u;
                        M.mask = mask;
                        M.flags = 1;
                        M.t.tau = J.tau;
                        M.t.outA = J.table + (int64_t)l * slab + (int64_t)(vt * kPairVB) * rowlen + (int64_t)p_lo * NMP;
                        M.t.flA = J.rowflag + (size_t)l * J.n_v;
                        M.t.v0A = vt * kPairVB;
                        M.t.v0B = vt * kPairVB - delta;
                        M.slab = slab;
                        M.rowlen = (int32_t)rowlen;
                        M.n_v = J.n_v;
                        M.hasB = hasB ? 1 : 0;
                        sref[s] = kPairRows;
                        mbar_arrive(full0 + 8 * s);
                    }
                }
                push(act, mask, ent);
                const int adv = min(round, stages - r0);
                sl += adv;
                if (sl >= nsl) { sl -= nsl; wraps++; }
            }
        }
        {                                                  // terminate every row
            const bool act = lane == 0;
            uint32_t ent = 0;
            if (act) {
                if (wraps > 0) mbar_wait(empty0 + 8 * sl, (uint32_t)((wraps - 1) & 1));
                meta[sl].flags = 4;
                sref[sl] = kPairRows;
                ent = (uint32_t)sl | (uint32_t)(wraps & 1) << 7;
                mbar_arrive(full0 + 8 * sl);
            }
            push(act, (1u << kPairRows) - 1u, ent);
        }
        return;
    }

    // =============================================================== consumer warps
    const int r = warp;                                    // output row of the tile
    const bool isB = r >= kPairVB;
    constexpr int G8 = C >= 8 ? 1 : 8 / C;                 // lanes sharing a 128-byte window
    constexpr int RM = C >= 8 ? 8 : C;
    const int rot = (lane / G8) % RM;                      // lane + 32 has the same rotation
    double b0[NMP], b1[NMP];
#pragma unroll
    for (int i = 0; i < NMP; i++) { b0[i] = MP_INF; b1[i] = MP_INF; }
    int head = 0;
    for (;;) {
        while (vtail[r] == head) { }
        const uint32_t ent = reinterpret_cast<volatile uint8_t *>(rq[r])[head & (QN - 1)];
        head++;
        const int s = (int)(ent & 63u);
        mbar_wait(full0 + 8 * s, (ent >> 7) & 1u);
        const PairMeta &M = meta[s];
        const int flags = M.flags;
        if (flags & 4) break;
        const int np = M.np, n_m = M.n_m;
        if (flags & 1) {                                   // tile end: clamp (Q12), store, flag
            const int v = isB ? M.t.v0B + (r - kPairVB) : M.t.v0A + r;
            const bool ok = (!isB || M.hasB) && v >= 0 && v < M.n_v;
            bool fin = false;
            if (ok) {
                double *o = M.t.outA + (int64_t)(v - M.t.v0A) * M.rowlen + (isB ? M.slab : (int64_t)0);
                if (lane < np) fin |= pair_store<NMP>(b0, o + (int64_t)lane * NMP, rot, M.t.tau, n_m);
                if (lane + 32 < np) fin |= pair_store<NMP>(b1, o + (int64_t)(lane + 32) * NMP, rot, M.t.tau, n_m);
            }
            if (__ballot_sync(0xffffffffu, fin) && lane == 0)
                atomicOr(M.t.flA + (isB ? M.n_v : 0) + v, 1u);
#pragma unroll
            for (int i = 0; i < NMP; i++) { b0[i] = MP_INF; b1[i] = MP_INF; }
        } else {
            const uint32_t code = M.e.code[r];
            const int d = (int)(code & 127u);
            const bool nf = (code >> 7) & 1u;
            const double U = isB ? M.e.U1 : M.e.U0;
            const double *base = ring + (size_t)s * seg_doubles;
            if (lane < np) pair_relax<NMP>(b0, base + lane * NMP, rot, d, nf, U, n_m);
            if (lane + 32 < np) pair_relax<NMP>(b1, base + (lane + 32) * NMP, rot, d, nf, U, n_m);
        }
        __syncwarp();
        if (lane == 0) {
            __threadfence_block();
            if (atomicSub(&sref[s], 1) == 1) mbar_arrive(empty0 + 8 * s);
        }
    }
}

// ---------------------------------------------------------------------------
// Option k = l1 of layer l1 (= l+1 of the pair): N and S from slab l1-1, which
// the pair pass has just completed.  One warp per (job, v).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(128) pair_fixup_kernel(const Job *jobs, int l1, int nmp) {
    __shared__ Job sJ;
    if (threadIdx.x < sizeof(Job) / 8)
        reinterpret_cast<uint64_t *>(&sJ)[threadIdx.x] =
            __ldg(reinterpret_cast<const uint64_t *>(jobs + blockIdx.y) + threadIdx.x);
    __syncthreads();
    const Job &J = sJ;
    if (l1 > J.L || J.P < 2) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int v = blockIdx.x * 4 + warp;
    if (v >= J.n_v) return;
    const int k = l1;
    if (k < J.kwin[l1]) return;                  // U(l1,l1) > tau or its weights do not fit
    const double U = __dsub_rn(J.Up[l1], J.Up[l1 - 1]);
    int64_t d;
    const int32_t tr = transition(J, k, l1, v, U, &d);
    if (tr < 0) return;
    const unsigned long long per = (unsigned long long)(J.P - 1) * (unsigned long long)J.n_m;
    const int vn = tr & 0xFFFF;
    const bool nf = (tr >> 24) & 1;
    const bool use = J.rowflag[(size_t)(k - 1) * J.n_v + vn] != 0u;
    if (lane == 0) {
        atomicAdd(J.eff, per);
        if (use) atomicAdd(J.useful, per);
    }
    if (!use) return;
    const size_t rowlen = (size_t)J.P * nmp;
    const size_t slab = (size_t)J.n_v * rowlen;
    double *row = J.table + (size_t)l1 * slab + (size_t)v * rowlen;
    const double *src = J.table + (size_t)(k - 1) * slab + (size_t)vn * rowlen;
    const double tau = J.tau;
    bool fin = false;
    for (int c = nmp + lane; c < J.P * nmp; c += 32) {       // cells p >= 1
        const int m = c & (nmp - 1);
        if (m >= J.n_m) continue;
        double b = row[c];
        if (nf) b = dmin(b, src[c - nmp]);                    // N
        if ((int64_t)m + d <= (int64_t)(J.n_m - 1))           // S
            b = dmin(b, __dadd_rn(U, src[c + d]));
        b = b <= tau ? b : MP_INF;                            // clamp (Q12)
        row[c] = b;
        fin |= b <= tau;
    }
    if (__ballot_sync(0xffffffffu, fin) && lane == 0) atomicOr(J.rowflag + (size_t)l1 * J.n_v + v, 1u);
}

// tile geometry of the pair path: (v-tiles incl. kPairE extra) x p-tiles of <= 64 rows
void pair_geom(int P, int n_v, int *np, int *n_ptiles, int *n_vtiles, int *n_tiles) {
    const int rows = P - 1 > 0 ? P - 1 : 1;
    *np = rows < kPairNp ? rows : kPairNp;
    *n_ptiles = (rows + *np - 1) / *np;
    *n_vtiles = (n_v + kPairVB - 1) / kPairVB + kPairE;
    *n_tiles = *n_vtiles * *n_ptiles;
}

int pair_list_cap(int max_L) { return kPairRows * (max_L > 0 ? max_L : 1); }
size_t pair_entry_bytes() { return sizeof(PairEntry); }

// ring slots: as many as fit in ~200 KB
int pair_nsl(int np, int nmp) {
    const int seg = (np + 1) * nmp * 8;
    int slots = (200 * 1024) / seg;
    return slots > kPairSlotsMax ? kPairSlotsMax : slots;
}

bool pair_supported(int P, int nmp) { return P >= 2 && (nmp == 4 || nmp == 8); }

void launch_pair_trans(const Job *jobs, int n_jobs, int n_v_max, int l, int nmp, size_t buf_off, size_t cnt_off,
                       cudaStream_t s) {
    const int nvt = (n_v_max + kPairVB - 1) / kPairVB + kPairE;
    pair_trans_kernel<<<dim3((nvt + 3) / 4, n_jobs), 128, 0, s>>>(jobs, l, nmp, buf_off, cnt_off);
}

void launch_pair_fixup(const Job *jobs, int n_jobs, int n_v_max, int l1, int nmp, cudaStream_t s) {
    pair_fixup_kernel<<<dim3((n_v_max + 3) / 4, n_jobs), 128, 0, s>>>(jobs, l1, nmp);
}

void launch_pair_step(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp, int np, int nsl,
                      int grid, size_t buf_off, size_t cnt_off, cudaStream_t s) {
    const int smem = nsl * (np + 1) * nmp * 8;
    int round = nsl / 2;
    if (round > 32) round = 32;
    if (round < 1) round = 1;
    switch (nmp) {
#define MP_CASE(N)                                                                                     \
    case N:                                                                                            \
        cudaFuncSetAttribute(pair_step_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);   \
        pair_step_kernel<N><<<grid, kPairThreads, smem, s>>>(jobs, tile_job, n_tiles, l, np, nsl, round, buf_off, cnt_off); \
        break;
        MP_CASE(4) MP_CASE(8)
#undef MP_CASE
    }
}

}  // namespace mp
