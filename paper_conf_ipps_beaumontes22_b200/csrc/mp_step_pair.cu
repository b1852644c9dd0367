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
#include <cstdlib>
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
__device__ __forceinline__ void mbar_arrive_cnt(uint32_t bar, uint32_t cnt) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(cnt) : "memory");
}
// Row queues inside one CTA: a queue entry is ONE 32-bit shared word that carries its
// own wrap bit (bit 31 = ((position / QN) & 1) ^ 1; the queue starts zeroed), so the
// consumer polls the entry itself.  No second location (a tail) is published, hence
// no cross-location ordering is needed: single-location coherence of the producer's
// volatile store and the consumer's volatile load is all the handoff relies on.  The
// slot's data and metadata are ordered by the slot's full mbarrier (arrive = release,
// try_wait = acquire; the bulk copy completes on it), not by the queue word.
// MP_QUEUE_ATOMIC=1: the same handoff through shared-memory atomics (exchange / or 0),
// which compute-sanitizer racecheck recognises as synchronising (A/B variant).
#ifndef MP_QUEUE_ATOMIC
#define MP_QUEUE_ATOMIC 0
#endif
__device__ __forceinline__ void st_entry_s(uint32_t saddr, uint32_t v) {   // shared-window address
#if MP_QUEUE_ATOMIC
    asm volatile("atom.shared::cta.exch.b32 _, [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
#else
    asm volatile("st.volatile.shared::cta.u32 [%0], %1;" ::"r"(saddr), "r"(v));
#endif
}
__device__ __forceinline__ uint32_t ld_entry(const uint32_t *p) {
    uint32_t v;
#if MP_QUEUE_ATOMIC
    asm volatile("atom.shared::cta.or.b32 %0, [%1], 0;" : "=r"(v) : "r"(smem_u32(p)) : "memory");
#else
    asm volatile("ld.volatile.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
#endif
    return v;
}

}  // namespace

#ifndef MP_PAIR_VB
#define MP_PAIR_VB 4
#endif
constexpr int kPairVB = MP_PAIR_VB;              // delay rows per layer in a tile
constexpr int kPairRows = 2 * kPairVB;           // output rows (= consumer warps) per tile
constexpr int kPairE = 16 / kPairVB;             // extra v-tiles: layer l+1 rows are shifted by <= 16 levels
#ifndef MP_PAIR_CTAS
#define MP_PAIR_CTAS (8 / MP_PAIR_VB)
#endif
constexpr int kPairCtas = MP_PAIR_CTAS;           // resident CTAs per SM (one producer warp each)
constexpr int kPairNp = 64;                      // processor rows per tile (2 per consumer thread)
constexpr int kPairSlotsMax = kPairVB > 4 ? 48 : 32;  // ring slots (6-bit slot index in the queue word)
#ifndef MP_PAIR_NPROD
#define MP_PAIR_NPROD 1
#endif
constexpr int kPairProd = MP_PAIR_NPROD;         // producer warps: producer p takes the CTA's tiles p, p+2, ..
                                                 // with its own half of the ring and its own row queues
constexpr int kPairThreads = 32 * (kPairRows + kPairProd);
constexpr int kPairHdr = 2;                      // header entries at the head of each tile list
#ifndef MP_POLL_NS
#define MP_POLL_NS 250
#endif
#ifndef MP_PAIR_PROF
#define MP_PAIR_PROF 0                                     // 1: MADPIPE_PROF=1 cycle counters in pair_step_kernel (build variant "prof")
#endif
#ifndef MP_PAIR_L2PF
#define MP_PAIR_L2PF 3                                     // list entries prefetched into L2, in producer rounds
#endif
#ifndef MP_PAIR_ONEROW
#define MP_PAIR_ONEROW 1                                   // one processor row per thread for tiles of <= 32
#endif
#ifndef MP_DIAG
#define MP_DIAG 0                                          // 1: the `diag` launch argument is honoured (diagnostic
#endif                                                     // replays only, wrong results): bit 0 = consumers skip
                                                           // the relaxation, bit 1 = producer skips the copies
#ifndef MP_PAIR_STAGE
#define MP_PAIR_STAGE 32
#endif
constexpr int kPairStage = MP_PAIR_STAGE;        // list head (header + entries) prefetched per tile

// One source row of a tile's merged list (pair_trans_kernel -> pair_step_kernel).
struct PairEntry {
    uint16_t k;        // option k: the source is slab k-1
    uint16_t vp;       // next delay level v' (source row)
    uint16_t mask;     // output rows of the tile that read it (bit r: r < kPairVB layer l, else l+1)
    uint16_t pad;
    uint8_t code[kPairRows];   // per row r: d (bits 0-6, clamped to 127) | nf << 7
    double U0, U1;     // U(k,l), U(k,l+1)
};
static_assert(sizeof(PairEntry) == 24 + kPairRows, "PairEntry size");

// Tile header (the first kPairHdr entries of a tile list): what the producer
// needs for the tile without reading the job descriptor.  n < 0: the job has no
// layer l (l > L in a batch of chains of different lengths): the tile is skipped.
struct PairHdr {
    int32_t n;         // entries
    int32_t l;         // first layer of the pair
    int32_t hasB;      // l+1 <= L
    int32_t n_m;
    double tau;
    double *table;     // the job's DP table
    uint32_t *flA;     // rowflag + l * n_v
    int32_t n_v, P;
    int32_t v0A, v0B;  // first delay row of layer l / layer l+1 in the tile
    int64_t pad_[1 + (kPairHdr * (24 + kPairRows) - 64) / 8];
};
static_assert(sizeof(PairHdr) == kPairHdr * sizeof(PairEntry), "PairHdr size");

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
__device__ __forceinline__ void pair_trans_body(const Job &J, int vt, int lane, int l, int nmp, size_t buf_off,
                                                int fix_slab, int unv_from) {
    // unv_from: source slabs >= unv_from are still being written by the step (and fixup)
    // kernels of the previous pass when this launch overlaps them (MADPIPE_TRANS_OVERLAP):
    // their row flags are not consulted and every live entry reading them is kept (a
    // superset of the useful ones, so the skip stays exact).
    // fix_slab (= l-1, or -1): this launch runs concurrently with pair_fixup_kernel of
    // slab fix_slab, which may still turn that slab's row flags on.  For a source row w
    // of that slab whose flag is still 0, the entry is kept if the fixup could make the
    // row finite -- its option k = fix_slab is live and reads a row of slab fix_slab-1
    // that holds a finite value -- a superset of what the fixup will flag, so the skip
    // stays exact.
    constexpr int KG = 32 / kPairRows;           // k values per warp iteration
    if (vt >= pair_vtiles(J.n_v)) return;
    if (l > J.L) {                               // no layer l (a shorter chain of the batch):
        if (lane == 0)                           // the step kernel skips the tile
            reinterpret_cast<PairHdr *>(reinterpret_cast<PairEntry *>(J.tlist) + buf_off +
                                        (size_t)vt * J.code_cap)->n = -1;
        return;
    }
    const bool hasB = l + 1 <= J.L;
    const int delta = pair_shift(J, l);
    const int r = lane % kPairRows, h = lane / kPairRows;   // row r of the tile; lane group h takes k = kb + h
    const bool isB = r >= kPairVB;
    const int lr = isB ? l + 1 : l;              // the row's layer
    const int v = isB ? vt * kPairVB - delta + (r - kPairVB) : vt * kPairVB + r;
    const bool row_ok = (!isB || hasB) && v >= 0 && v < J.n_v;
    if (__ballot_sync(0xffffffffu, row_ok) == 0u) {    // no output row in this tile (one of the extra v-tiles
        if (lane == 0)                           // beyond the layer-(l+1) shift): the step kernel skips it
            reinterpret_cast<PairHdr *>(reinterpret_cast<PairEntry *>(J.tlist) + buf_off +
                                        (size_t)vt * J.code_cap)->n = -1;
        return;
    }
    const size_t rowlen = (size_t)J.P * nmp;
    const size_t slab = (size_t)J.n_v * rowlen;
    const double Ulr = J.Up[lr];
    const double Ul = J.Up[l], Ul1 = hasB ? J.Up[l + 1] : 0.0;
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
    const RowCtx rc = row_ctx(J, row_ok ? v : 0);    // the row's k-invariant part of every transition
    // option k = l+1 of the layer-(l+1) rows, for pair_fixup_kernel: its transition
    // (or kSkip), one word per row, buffer (pass % 2) -- the fixup of this pass runs
    // while the next pass's lists are built
    if (isB && row_ok && h == 0) {
        int32_t fx = kSkip;
        if (l + 1 >= kw) {
            int64_t d;
            fx = transition_rc(J, l + 1, l + 1, rc, __dsub_rn(Ul1, Ul), &d);
        }
        J.codes[(size_t)((l >> 1) & 1) * J.n_v + v] = fx;
    }
    int n = 0;
    PairEntry *tl = reinterpret_cast<PairEntry *>(J.tlist) + buf_off + (size_t)vt * J.code_cap;
    PairEntry *list = tl + kPairHdr;
    const unsigned gmask = ((1u << kPairRows) - 1u) << (h * kPairRows);
    // k <= l: sources in slabs <= l-1 (final).  TU k-groups per chunk: their transitions
    // (independent global loads) and then their row flags are fetched together, so a
    // chunk costs two memory round trips instead of two per k-group.
#ifndef MP_TRANS_TU
#define MP_TRANS_TU 1
#endif
    constexpr int TU = MP_TRANS_TU;
    for (int kc = kA; kc <= l; kc += KG * TU) {
        int key[TU];
        uint32_t code[TU];
#pragma unroll
        for (int u = 0; u < TU; u++) {
            const int k = kc + u * KG + h;
            key[u] = -1 - lane;                  // unique unless the row reads a source
            code[u] = 0;
            if (row_ok && k <= l && k >= kw) {
                int64_t d;
                const int32_t tr = transition_rc(J, k, lr, rc, __dsub_rn(Ulr, J.Up[k - 1]), &d);
                if (tr >= 0) {
                    live++;
                    key[u] = (k << 16) | (tr & 0xFFFF);
                    code[u] = (uint32_t)(d > 127 ? 127 : d) | ((tr >> 24) & 1u) << 7;
                }
            }
        }
        uint32_t fl[TU];
#pragma unroll
        for (int u = 0; u < TU; u++) {
            const int k = key[u] >> 16;
            fl[u] = 1u;
            if (key[u] >= 0) fl[u] = J.rowflag[(size_t)(k - 1) * J.n_v + (key[u] & 0xFFFF)];
        }
#pragma unroll
        for (int u = 0; u < TU; u++) {
            const int sk = (key[u] >> 16) - 1;   // source slab
            if (key[u] >= 0 && sk >= unv_from) fl[u] = 1u;
            if (key[u] >= 0 && fl[u] == 0u && sk == fix_slab && sk >= J.kwin[sk]) {
                const int w = key[u] & 0xFFFF;
                int64_t d2;
                const int32_t t2 = transition(J, sk, sk, w, __dsub_rn(J.Up[sk], J.Up[sk - 1]), &d2);
                if (t2 >= 0 && J.rowflag[(size_t)(sk - 1) * J.n_v + (t2 & 0xFFFF)] != 0u) fl[u] = 1u;
            }
        }
#pragma unroll
        for (int u = 0; u < TU; u++) {
            // a source row that is +inf everywhere contributes +inf (exact skip)
            if (key[u] >= 0 && fl[u] == 0u) key[u] = -1 - lane;
            if (key[u] >= 0) useful++;
            const unsigned grp = __match_any_sync(0xffffffffu, key[u]);
            const int leader = __ffs(grp) - 1;
            const bool lead = key[u] >= 0 && leader == lane;
            const unsigned lb = __ballot_sync(0xffffffffu, lead);
            int idx = n + __popc(lb & ((1u << lane) - 1u));
            idx = __shfl_sync(0xffffffffu, idx, leader);
            if (lead) {
                const int k = key[u] >> 16;
                PairEntry *e = list + idx;
                const double Uk = J.Up[k - 1];
                *reinterpret_cast<uint64_t *>(e) = (uint64_t)(uint32_t)k | (uint64_t)(uint32_t)(key[u] & 0xFFFF) << 16 |
                                                   (uint64_t)((grp & gmask) >> (h * kPairRows)) << 32;
                e->U0 = __dsub_rn(Ul, Uk);
                e->U1 = hasB ? __dsub_rn(Ul1, Uk) : 0.0;
            }
            if (key[u] >= 0) list[idx].code[r] = (uint8_t)code[u];
            n += __popc(lb);
        }
    }
    if (lane == 0) {
        PairHdr hd;
        hd.n = n;
        hd.l = l;
        hd.hasB = hasB ? 1 : 0;
        hd.n_m = J.n_m;
        hd.tau = J.tau;
        hd.table = J.table;
        hd.flA = J.rowflag + (size_t)l * J.n_v;
        hd.n_v = J.n_v;
        hd.P = J.P;
        hd.v0A = vt * kPairVB;
        hd.v0B = vt * kPairVB - delta;
        for (auto &x : hd.pad_) x = 0;
        *reinterpret_cast<PairHdr *>(tl) = hd;
    }
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

#ifndef MP_TRANS_MINB
#define MP_TRANS_MINB 8
#endif
__global__ void __launch_bounds__(128, MP_TRANS_MINB) pair_trans_kernel(const Job *jobs, int l, int nmp, size_t buf_off,
                                                         int fix_slab, int unv_from, int xb, int n_items) {
    // block item = (job, group of 4 v-tiles); a grid of n_items blocks takes one item each,
    // a smaller (persistent) grid loops over them so that the fixup kernel's blocks can run
    // beside it
    __shared__ Job sJ;
    for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
        const int job = it / xb, bx = it - job * xb;
        __syncthreads();
        if (threadIdx.x < sizeof(Job) / 8)
            reinterpret_cast<uint64_t *>(&sJ)[threadIdx.x] =
                __ldg(reinterpret_cast<const uint64_t *>(jobs + job) + threadIdx.x);
        __syncthreads();
        pair_trans_body(sJ, bx * 4 + (threadIdx.x >> 5), threadIdx.x & 31, l, nmp, buf_off, fix_slab, unv_from);
    }
}

// ---------------------------------------------------------------------------
// a5 for the layer pair: the persistent two-layer step kernel.
// ---------------------------------------------------------------------------
struct PairMeta {
    int16_t flags;          // 0 = data, 1 = tile end (store the rows), 4 = terminate
    int16_t np;             // processor rows of the tile
    int32_t n_m;
    union {
        struct { double U0, U1; uint8_t code[kPairRows]; } e;       // data: U(k,l), U(k,l+1), codes
        struct { double tau; double *outA; uint32_t *flA; int32_t v0A, v0B; } t;  // tile end
    };
    int64_t slab;           // doubles per slab
    int32_t rowlen, n_v;
    int32_t hasB, pad_;
};
static_assert(sizeof(PairMeta) == 64, "PairMeta size");

// relax one processor row of NMP levels held in lane-rotated chunk order (the
// layout of step_persist_kernel's ROW mode: chunk c of a thread holds levels
// 2j, 2j+1 with j = (c + rot) mod C, so a quarter-warp's 16-byte loads hit 8
// distinct bank groups).  `off[c]` = byte offset of the thread's source row p-1,
// chunk j, in the slot (precomputed once); S reads row p, levels m + d: the same
// offset + NMP*8 + 8d.  S candidates with m + d > n_m - 1 are read (in bounds of
// the padded ring) and discarded by predicate, so the code has no per-lane branch.
// S candidates of one slot: b = (valid && U + src[m+d] < b) ? U + src[m+d] : b, the
// validity folded into the compare (one DSETP with a predicate operand and one 64-bit
// select per level).  ODD: d is odd, so the shifted levels are not 16-byte aligned.
template <int NMP, bool TWO, bool ODD>
__device__ __forceinline__ void pair_relax_s(double (&b0)[NMP], double (&b1)[NMP], const char *srow,
                                             const int (&off0)[NMP / 2], const int (&off1)[NMP / 2],
                                             const int (&m2)[NMP / 2], double U, int lim) {
    constexpr int C = NMP / 2;
#pragma unroll
    for (int c = 0; c < C; c++) {
        const bool v0 = m2[c] <= lim, v1 = m2[c] + 1 <= lim;
        double y0, y1, z0 = 0.0, z1 = 0.0;
        if (!ODD) {
            const double2 y = *reinterpret_cast<const double2 *>(srow + off0[c]);
            y0 = y.x; y1 = y.y;
            if (TWO) {
                const double2 z = *reinterpret_cast<const double2 *>(srow + off1[c]);
                z0 = z.x; z1 = z.y;
            }
        } else {
            y0 = *reinterpret_cast<const double *>(srow + off0[c]);
            y1 = *reinterpret_cast<const double *>(srow + off0[c] + 8);
            if (TWO) {
                z0 = *reinterpret_cast<const double *>(srow + off1[c]);
                z1 = *reinterpret_cast<const double *>(srow + off1[c] + 8);
            }
        }
        const double c0 = __dadd_rn(U, y0), c1 = __dadd_rn(U, y1);
        asm("{\n\t.reg .pred q0, q1, p;\n\t"
            "setp.ne.u32 q0, %4, 0;\n\t"
            "setp.ne.u32 q1, %5, 0;\n\t"
            "setp.lt.and.f64 p, %2, %0, q0;\n\t"
            "selp.f64 %0, %2, %0, p;\n\t"
            "setp.lt.and.f64 p, %3, %1, q1;\n\t"
            "selp.f64 %1, %3, %1, p;\n\t}"
            : "+d"(b0[2 * c]), "+d"(b0[2 * c + 1])
            : "d"(c0), "d"(c1), "r"((unsigned)v0), "r"((unsigned)v1));
        if (TWO) {
            const double e0 = __dadd_rn(U, z0), e1 = __dadd_rn(U, z1);
            asm("{\n\t.reg .pred q0, q1, p;\n\t"
                "setp.ne.u32 q0, %4, 0;\n\t"
                "setp.ne.u32 q1, %5, 0;\n\t"
                "setp.lt.and.f64 p, %2, %0, q0;\n\t"
                "selp.f64 %0, %2, %0, p;\n\t"
                "setp.lt.and.f64 p, %3, %1, q1;\n\t"
                "selp.f64 %1, %3, %1, p;\n\t}"
                : "+d"(b1[2 * c]), "+d"(b1[2 * c + 1])
                : "d"(e0), "d"(e1), "r"((unsigned)v0), "r"((unsigned)v1));
        }
    }
}

template <int NMP, bool TWO>
__device__ __forceinline__ void pair_relax(double (&b0)[NMP], double (&b1)[NMP], const char *slot,
                                           const int (&off0)[NMP / 2], const int (&off1)[NMP / 2],
                                           const int (&m2)[NMP / 2], int d, bool nf, double U, int lim) {
    // both processor rows of the thread at once (TWO; one row when the tile has <= 32
    // processor rows): the S validity predicates (which depend on the lane's chunk
    // rotation, not on the row) are formed once per chunk, and each is folded into the
    // candidate's compare (one DSETP with a predicate operand and one 64-bit select per
    // level, rather than a second select for the predicate)
    constexpr int C = NMP / 2;
    if (nf) {                                                    // N
#pragma unroll
        for (int c = 0; c < C; c++) {
            const double2 x = *reinterpret_cast<const double2 *>(slot + off0[c]);
            b0[2 * c] = dmin(b0[2 * c], x.x);
            b0[2 * c + 1] = dmin(b0[2 * c + 1], x.y);
            if (TWO) {
                const double2 y = *reinterpret_cast<const double2 *>(slot + off1[c]);
                b1[2 * c] = dmin(b1[2 * c], y.x);
                b1[2 * c + 1] = dmin(b1[2 * c + 1], y.y);
            }
        }
    }
    if (lim >= 0) {                                              // S: valid iff m <= lim = n_m-1-d
        // the level shift d is the same for the whole warp: one branch on its parity, so each
        // path issues only its own loads (16-byte pairs for even d, 8-byte singles for odd d)
        const char *srow = slot + NMP * 8 + 8 * d;
        if (d & 1) pair_relax_s<NMP, TWO, true>(b0, b1, srow, off0, off1, m2, U, lim);
        else pair_relax_s<NMP, TWO, false>(b0, b1, srow, off0, off1, m2, U, lim);
    }
}

// clamp (Q12) and store one processor row; returns whether a value is finite
template <int NMP>
__device__ __forceinline__ bool pair_store(const double (&best)[NMP], double *o, int rot, double tau, int n_m) {
    constexpr int C = NMP / 2;
    bool fin = false;
    unsigned any = 0u;
#pragma unroll
    for (int c = 0; c < C; c++) {
        const int j = (c + rot) & (C - 1);
        double2 r;
        // r = (level exists && b <= tau) ? b : +inf; any |= that predicate
        asm("{\n\t.reg .pred q0, q1, p0, p1;\n\t"
            "setp.lt.s32 q0, %6, %7;\n\t"
            "setp.lt.s32 q1, %8, %7;\n\t"
            "setp.le.and.f64 p0, %3, %5, q0;\n\t"
            "setp.le.and.f64 p1, %4, %5, q1;\n\t"
            "selp.f64 %0, %3, 0d7FF0000000000000, p0;\n\t"
            "selp.f64 %1, %4, 0d7FF0000000000000, p1;\n\t"
            "@p0 or.b32 %2, %2, 1;\n\t"
            "@p1 or.b32 %2, %2, 1;\n\t}"
            : "=d"(r.x), "=d"(r.y), "+r"(any)
            : "d"(best[2 * c]), "d"(best[2 * c + 1]), "d"(tau), "r"(2 * j), "r"(n_m), "r"(2 * j + 1));
        *reinterpret_cast<double2 *>(o + 2 * j) = r;
    }
    fin = any != 0u;
    return fin;
}

template <int NMP>
__global__ void __launch_bounds__(kPairThreads, kPairCtas) pair_step_kernel(const int2 *__restrict__ tdesc, int n_tiles,
                                                                    const PairEntry *__restrict__ lists,
                                                                    int np_max, int nsl, int round,
                                                                    int stage_n, unsigned long long *prof,
                                                                    int diag) {
#if !MP_DIAG
    diag = 0;                                              // MADPIPE_REPLAY diagnostics compiled out
#endif
    // Slots are shared by the rows that read them: the producer pushes each slot
    // (with the parity of its full-barrier phase) into the queue of every row in
    // its mask; a row warp visits only its own slots; the last reader (reference
    // count) releases the slot's empty barrier.  Tile ends and the final
    // termination are slots without data pushed to all rows.  tdesc[tile] =
    // (offset of the tile's list in `lists`, processor tile).
#if !MP_PAIR_PROF
    prof = nullptr;                                        // cycle counters compiled out (MADPIPE_PROF reads zeros)
#endif
    constexpr int C = NMP / 2;
    constexpr int QN = kPairSlotsMax > 32 ? 64 : 32;       // queue entries per row (>= slots, power of 2)
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ __align__(8) uint64_t full[kPairSlotsMax];
    __shared__ __align__(8) uint64_t empty[kPairSlotsMax];
    __shared__ __align__(16) PairMeta meta[kPairSlotsMax];
    // per-row queues: slot | parity << 6 | control << 7 | n_m << 8 | two rows << 12 | code << 16 | wrap bit << 31
    __shared__ uint32_t rq[kPairProd][kPairRows][QN];
    __shared__ __align__(128) PairEntry stage[kPairProd][2][kPairStage];   // list heads of this and the next tile
    __shared__ __align__(8) uint64_t stbar[kPairProd][2];

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int seg_doubles = (np_max + 1) * NMP;
    const uint32_t full0 = smem_u32(&full[0]), empty0 = smem_u32(&empty[0]);
    const uint32_t ring_s = smem_u32(dsm);
    if (tid == 0) {
        for (int s = 0; s < nsl; s++) {
            mbar_init(full0 + 8 * s, 1);
            mbar_init(empty0 + 8 * s, kPairRows);
        }
        for (int p = 0; p < kPairProd; p++) {
            mbar_init(smem_u32(&stbar[p][0]), 1);
            mbar_init(smem_u32(&stbar[p][1]), 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    for (int i = tid; i < kPairProd * kPairRows * QN; i += blockDim.x) (&rq[0][0][0])[i] = 0u;
    __syncthreads();

    if (warp >= kPairRows) {
        // =========================================================== producer warp(s)
        const int pw = warp - kPairRows;                   // producer index
        const int nslp = nsl / kPairProd, s_base = pw * nslp;   // this producer's ring slots
        int sl = 0, wraps = 0;
        int tails[kPairRows];                              // entries pushed per row (same in every lane)
#pragma unroll
        for (int rr = 0; rr < kPairRows; rr++) tails[rr] = 0;
        const unsigned lt = (1u << lane) - 1u;
        const uint32_t rq_s = smem_u32(&rq[pw][0][0]);     // shared address of this producer's queues
        auto push = [&](bool act, uint32_t mask, uint32_t ent, uint64_t codes, uint64_t codes_hi) {   // byte rr = row rr
            // append ent (+ the row's code, + the wrap bit of its position) to the queue of
            // every row in mask, in lane order.  All ballots first, then the positions and
            // words, then the stores: independent work the scheduler can overlap.
            unsigned bal[kPairRows];
#pragma unroll
            for (int rr = 0; rr < kPairRows; rr++) bal[rr] = __ballot_sync(0xffffffffu, act && ((mask >> rr) & 1u));
            uint32_t addr[kPairRows], word[kPairRows];
#pragma unroll
            for (int rr = 0; rr < kPairRows; rr++) {
                const int pos = tails[rr] + __popc(bal[rr] & lt);
                const uint64_t cw = rr < 8 ? codes : codes_hi;
                addr[rr] = rq_s + 4u * (uint32_t)(rr * QN + (pos & (QN - 1)));
                word[rr] = ent | (uint32_t)((cw >> (8 * (rr & 7))) & 0xFFu) << 16 | (uint32_t)(((pos / QN) & 1) ^ 1) << 31;
                tails[rr] += __popc(bal[rr]);
            }
#pragma unroll
            for (int rr = 0; rr < kPairRows; rr++)
                if ((bal[rr] >> lane) & 1u) st_entry_s(addr[rr], word[rr]);
        };
        // prof (MADPIPE_PROF=1): [0] producer cycles, [1] empty-barrier waits (max over lanes),
        // [2] tile setup (header), [3] consumer cycles, [4] queue waits, [5] full waits, [6] data
        // slots consumed (row visits), [7] tiles
        long long t_p0 = clock64(), t_we = 0, t_set = 0, n_tl = 0, t_push = 0;
        // the head of each tile's list (header + first entries) is bulk-copied into a
        // staging buffer one tile ahead, so a tile starts without a global-load round trip
        const uint32_t st0 = smem_u32(&stbar[pw][0]);
        const uint32_t stage_bytes = (uint32_t)stage_n * (uint32_t)sizeof(PairEntry);
        auto stage_copy = [&](int2 dsc, int buf) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive_expect_tx(st0 + 8 * buf, stage_bytes);
            bulk_g2s(smem_u32(&stage[pw][buf][0]), lists + dsc.x, stage_bytes, st0 + 8 * buf);
        };
        // with two producers both walk the same tiles and split each tile's entries (producer
        // pw takes entries pw, pw + 2, ...), each ending its share with a tile-end marker
        const int G = (int)gridDim.x;                       // tile stride
        const int t0 = (int)blockIdx.x;
        int2 desc = t0 < n_tiles ? __ldg(tdesc + t0) : make_int2(0, 0);
        int2 nextd = t0 + G < n_tiles ? __ldg(tdesc + t0 + G) : make_int2(0, 0);
        if (lane == 0 && t0 < n_tiles) stage_copy(desc, 0);
        int it = 0;
        for (int tile = t0; tile < n_tiles; tile += G, it++) {
            const long long t_t0 = prof ? clock64() : 0;
            const int buf = it & 1;
            if (lane == 0 && tile + G < n_tiles) stage_copy(nextd, buf ^ 1);
            const int2 mine = desc;
            desc = nextd;
            nextd = tile + 2 * G < n_tiles ? __ldg(tdesc + tile + 2 * G) : make_int2(0, 0);
            mbar_wait(st0 + 8 * buf, (uint32_t)((it >> 1) & 1));
            const PairEntry *tl = lists + mine.x;
            const PairEntry *sg = stage[pw][buf];
            const PairHdr hd = *reinterpret_cast<const PairHdr *>(sg);
            auto entry = [&](int e) -> PairEntry { return e + kPairHdr < stage_n ? sg[kPairHdr + e] : tl[kPairHdr + e]; };
            const int pt = mine.y;
            const int p_lo = 1 + pt * np_max;
            const int np = min(np_max, hd.P - p_lo);
            // a job with no layer l, a tile with no output row, or no processors in this tile:
            // nothing to store, no slot at all
            if (hd.n < 0 || np <= 0) continue;
            // first round's entries
            const int n_all = hd.n;
            const int n = (n_all - pw + kPairProd - 1) / kPairProd;   // this producer's share of the entries
            auto gidx = [&](int q_) { return q_ * kPairProd + pw; };   // share index -> list index
            PairEntry cur;
            if (n > 0 && lane < round && lane < n) cur = entry(gidx(lane));
            const int64_t rowlen = (int64_t)hd.P * NMP;
            const int64_t slab = (int64_t)hd.n_v * rowlen;
            const uint32_t seg_bytes = (uint32_t)(np + 1) * NMP * 8u;
            const int stages = n + 1;                      // entries, then the tile-end marker
            if (prof) { t_set += clock64() - t_t0; n_tl++; }
            for (int r0 = 0; r0 < stages; r0 += round) {
                const int q = r0 + lane;
                const bool act = lane < round && q < stages;
                PairEntry nxt;                             // prefetch the next round's entry
                if (lane < round && q + round < n) nxt = entry(gidx(q + round));
#if MP_PAIR_L2PF
                // and pull entries MP_PAIR_L2PF rounds ahead into L2 (lists beyond the staged head
                // are read from global memory; a DRAM miss there stalls the whole pipeline)
                {
                    const int qf = q + MP_PAIR_L2PF * round;
                    if (lane < round && qf < n && gidx(qf) + kPairHdr >= stage_n)
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(tl + kPairHdr + gidx(qf)));
                }
#endif
                uint32_t mask = 0, ent = 0;
                uint64_t codes = 0, codes_hi = 0;           // in registers (an array was spilled)
                if (act) {
                    int s = sl + lane, use = wraps;
                    if (s >= nslp) { s -= nslp; use++; }
                    s += s_base;
                    const long long tw = prof ? clock64() : 0;
                    if (use > 0) mbar_wait(empty0 + 8 * s, (uint32_t)((use - 1) & 1));
                    if (prof) {
                        const unsigned dw = (unsigned)(clock64() - tw);
                        const unsigned mx = __reduce_max_sync(__activemask(), dw);
                        if (lane == 0) t_we += mx;
                    }
                    // queue entry: slot | parity << 6 | control << 7 | n_m << 8 (n_m <= 8) | np > 32 << 12 |
                    // row code << 16
                    ent = (uint32_t)s | (uint32_t)(use & 1) << 6 | (uint32_t)hd.n_m << 8 | (np > 32 || !MP_PAIR_ONEROW ? 4096u : 0u);
                    PairMeta &M = meta[s];
                    if (q < n) {
                        if (!(diag & 2))
                            bulk_g2s(ring_s + 8u * (uint32_t)(s * seg_doubles),
                                     hd.table + (int64_t)(cur.k - 1) * slab + (int64_t)cur.vp * rowlen +
                                         (int64_t)(p_lo - 1) * NMP,
                                     seg_bytes, full0 + 8 * s);
                        mask = cur.mask;
                        M.e.U0 = cur.U0;
                        M.e.U1 = cur.U1;
                        static_assert(kPairRows == 8 || kPairRows == 16, "codes packing");
                        codes = *reinterpret_cast<const uint64_t *>(cur.code);
                        if (kPairRows > 8) codes_hi = *reinterpret_cast<const uint64_t *>(cur.code + 8);
                        // rows that do not read the slot release it now
                        if (__popc(mask) < kPairRows) mbar_arrive_cnt(empty0 + 8 * s, kPairRows - __popc(mask));
                        if (diag & 2) mbar_arrive(full0 + 8 * s);
                        else mbar_arrive_expect_tx(full0 + 8 * s, seg_bytes);
                    } else {
                        mask = (1u << kPairRows) - 1u;
                        ent |= 128u;                       // control slot
                        M.np = (int16_t)np;
                        M.n_m = hd.n_m;
                        M.flags = 1;
                        M.t.tau = hd.tau;
                        M.t.flA = hd.flA;
                        M.slab = slab;
                        M.rowlen = (int32_t)rowlen;
                        M.n_v = hd.n_v;
                        M.hasB = hd.hasB;
                        M.t.v0A = hd.v0A;
                        M.t.v0B = hd.v0B;
                        M.t.outA = hd.table + (int64_t)hd.l * slab + (int64_t)hd.v0A * rowlen + (int64_t)p_lo * NMP;
                        mbar_arrive(full0 + 8 * s);
                    }
                }
                const long long tpu = prof ? clock64() : 0;
                push(act, mask, ent, codes, codes_hi);
                if (prof && lane == 0) t_push += clock64() - tpu;
                cur = nxt;
                const int adv = min(round, stages - r0);
                sl += adv;
                if (sl >= nslp) { sl -= nslp; wraps++; }
            }
        }
        {                                                  // terminate every row
            const bool act = lane == 0;
            uint32_t ent = 0;
            if (act) {
                const int sg_ = s_base + sl;
                if (wraps > 0) mbar_wait(empty0 + 8 * sg_, (uint32_t)((wraps - 1) & 1));
                meta[sg_].flags = 4;
                ent = (uint32_t)sg_ | (uint32_t)(wraps & 1) << 6 | 128u;   // control slot
                mbar_arrive(full0 + 8 * sg_);
            }
            push(act, (1u << kPairRows) - 1u, ent, 0ull, 0ull);
        }
        if (prof && lane == 0) {
            atomicAdd(prof + 0, (unsigned long long)(clock64() - t_p0));
            atomicAdd(prof + 1, (unsigned long long)t_we);
            atomicAdd(prof + 2, (unsigned long long)t_set);
            atomicAdd(prof + 7, (unsigned long long)n_tl);
            atomicAdd(prof + 8, (unsigned long long)t_push);
        }
        return;
    }
    // =============================================================== consumer warps
    const int r = warp;                                    // output row of the tile
    const bool isB = r >= kPairVB;
    constexpr int G8 = C >= 8 ? 1 : 8 / C;                 // lanes sharing a 128-byte window
    constexpr int RM = C >= 8 ? 8 : C;
    const int rot = (lane / G8) % RM;                      // lane + 32 has the same rotation
    int off0[C], off1[C], m2[C];                           // chunk offsets of rows lane, lane+32
#pragma unroll
    for (int c = 0; c < C; c++) {
        const int jj = (c + rot) & (C - 1);
        m2[c] = 2 * jj;
        off0[c] = (lane * NMP + 2 * jj) * 8;
        off1[c] = ((lane + 32) * NMP + 2 * jj) * 8;
    }
    double b0[NMP], b1[NMP];
#pragma unroll
    for (int i = 0; i < NMP; i++) { b0[i] = MP_INF; b1[i] = MP_INF; }
    const char *ring = reinterpret_cast<const char *>(dsm);
    const int seg_bytes = seg_doubles * 8;
    int head[kPairProd] = {};
    int qp = 0;                                            // the queue of the current tile's producer
    long long t_c0 = clock64(), t_q = 0, t_f = 0, n_sl = 0;
    for (;;) {
        const long long ta = prof ? clock64() : 0;
        // an empty queue (the entry still carries the previous wrap's bit): back off
        // instead of spinning (a spinning warp takes issue slots from the producer and
        // the working rows)
        const uint32_t want = (uint32_t)(((head[qp] / QN) & 1) ^ 1);
        const uint32_t *qe = &rq[qp][r][head[qp] & (QN - 1)];
        uint32_t ent;
        while (((ent = ld_entry(qe)) >> 31) != want) {
#if MP_POLL_NS > 0
            __nanosleep(MP_POLL_NS);
#endif
        }
        head[qp]++;
        const int s = (int)(ent & 63u);                    // this row's slot
        const long long tb = prof ? clock64() : 0;
        mbar_wait(full0 + 8 * s, (ent >> 6) & 1u);
        if (prof) { const long long tc = clock64(); t_q += tb - ta; t_f += tc - tb; n_sl++; }
        const PairMeta &M = meta[s];
        if (ent & 128u) {                                  // control slot (tile end / terminate)
        const int flags = M.flags;
        if ((flags & 4) && kPairProd > 1 && qp < kPairProd - 1) {
            qp++;                                          // the other producer's terminate follows
        } else if (flags & 4) {
            if (prof && lane == 0) {
                atomicAdd(prof + 3, (unsigned long long)(clock64() - t_c0));
                atomicAdd(prof + 4, (unsigned long long)t_q);
                atomicAdd(prof + 5, (unsigned long long)t_f);
                atomicAdd(prof + 6, (unsigned long long)n_sl);
            }
            break;
        }
        else if ((flags & 1) && kPairProd > 1 && qp < kPairProd - 1) {
            qp++;                                          // end of one producer's share of the tile
        } else if (flags & 1) {                            // tile end: clamp (Q12), store, flag
            const int np = M.np, n_m = M.n_m;
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
            qp = 0;                                        // the next tile starts with producer 0's share
        }
        } else {
            // rows lane and lane+32 are relaxed whether or not they exist in this tile
            // (np < 64): the extra rows read in-bounds ring bytes and are never stored
            const int d = (int)((ent >> 16) & 127u);
            const bool nf = (ent >> 23) & 1u;
            const double U = isB ? M.e.U1 : M.e.U0;
            const int lim = (int)((ent >> 8) & 15u) - 1 - d;   // n_m - 1 - d
            const char *slot = ring + s * seg_bytes;
            if (diag & 1) {
            } else if (ent & 4096u)                               // the tile has > 32 processor rows
                pair_relax<NMP, true>(b0, b1, slot, off0, off1, m2, d, nf, U, lim);
            else
                pair_relax<NMP, false>(b0, b1, slot, off0, off1, m2, d, nf, U, lim);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(empty0 + 8 * s);
    }
}

// ---------------------------------------------------------------------------
// Option k = l1 of layer l1 (= l+1 of the pair): N and S from slab l1-1, which
// the pair pass has just completed.  One warp per (job, v).
// ---------------------------------------------------------------------------
__device__ __forceinline__ void pair_fixup_body(const Job &J, int v, int lane, int l1, int nmp) {
    if (l1 > J.L || J.P < 2) return;
    if (v >= J.n_v) return;
    const int k = l1;
    // the transition of option k = l1 (pair_trans_body; kSkip if the window excludes it
    // or neither N nor S is possible)
    const int32_t tr = J.codes[(size_t)(((l1 - 1) >> 1) & 1) * J.n_v + v];
    if (tr < 0) return;
    const double U = __dsub_rn(J.Up[l1], J.Up[l1 - 1]);
    const int64_t d = (tr >> 16) & 0xFF;          // clamped to 255 (pack_trans): > n_m - 1 = no S
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
    double *__restrict__ row = J.table + (size_t)l1 * slab + (size_t)v * rowlen;
    const double *__restrict__ src = J.table + (size_t)(k - 1) * slab + (size_t)vn * rowlen;
    const double tau = J.tau;
    const int lim = J.n_m - 1 - (d > (int64_t)J.n_m ? J.n_m : (int)d);   // S valid iff m <= lim
    bool fin = false;
    // The row already holds the clamped min of the other options (values <= tau or
    // +inf); a cell is written back only when option k = l1 lowers it.  FB cells per
    // lane are loaded before any is stored (slab l1-1 is read-only here), so each warp
    // keeps FB loads in flight.
#ifndef MP_FIX_FB
#define MP_FIX_FB 4
#endif
    constexpr int FB = MP_FIX_FB;
    const int ncell = J.P * nmp;
    for (int c0 = nmp + lane; c0 < ncell; c0 += 32 * FB) {   // cells p >= 1
        double b0[FB], xn[FB], xs[FB];
#pragma unroll
        for (int i = 0; i < FB; i++) {
            const int c = c0 + 32 * i;
            const int m = c & (nmp - 1);
            const bool in = c < ncell && m < J.n_m;
            b0[i] = in ? row[c] : MP_INF;
            xn[i] = in && nf ? __ldg(src + c - nmp) : MP_INF;          // N
            xs[i] = in && m <= lim ? __ldg(src + c + d) : MP_INF;      // S
        }
#pragma unroll
        for (int i = 0; i < FB; i++) {
            const int c = c0 + 32 * i;
            double b = dmin(b0[i], xn[i]);
            if (xs[i] != MP_INF) b = dmin(b, __dadd_rn(U, xs[i]));
            b = b <= tau ? b : MP_INF;                        // clamp (Q12)
            if (b < b0[i]) row[c] = b;
            fin |= b <= tau;
        }
    }
    if (__ballot_sync(0xffffffffu, fin) && lane == 0) atomicOr(J.rowflag + (size_t)l1 * J.n_v + v, 1u);
}

#ifndef MP_FIX_MINB
#define MP_FIX_MINB 8
#endif
__global__ void __launch_bounds__(128, MP_FIX_MINB) pair_fixup_kernel(const Job *jobs, int l1, int nmp, int xb,
                                                                       int n_items) {
    __shared__ Job sJ;
    for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
        const int job = it / xb, bx = it - job * xb;
        __syncthreads();
        if (threadIdx.x < sizeof(Job) / 8)
            reinterpret_cast<uint64_t *>(&sJ)[threadIdx.x] =
                __ldg(reinterpret_cast<const uint64_t *>(jobs + job) + threadIdx.x);
        __syncthreads();
        pair_fixup_body(sJ, bx * 4 + (threadIdx.x >> 5), threadIdx.x & 31, l1, nmp);
    }
}


// tile geometry of the pair path: (v-tiles incl. kPairE extra) x p-tiles of <= 64 rows
void pair_geom(int P, int n_v, int *np, int *n_ptiles, int *n_vtiles, int *n_tiles) {
    const int rows = P - 1 > 0 ? P - 1 : 1;
    *np = rows < kPairNp ? rows : kPairNp;
    *n_ptiles = (rows + *np - 1) / *np;
    *n_vtiles = (n_v + kPairVB - 1) / kPairVB + kPairE;
    *n_tiles = *n_vtiles * *n_ptiles;
}

int pair_list_cap(int max_L) { return kPairHdr + kPairRows * (max_L > 0 ? max_L : 1); }
size_t pair_entry_bytes() { return sizeof(PairEntry); }

// ring slots per CTA (2 CTAs per SM): as many as fit in ~100 KB
int pair_nsl(int np, int nmp) {
    const int seg = (np + 1) * nmp * 8;
    int slots = ((kPairCtas > 2 ? 204 : 200) * 1024 / kPairCtas) / seg;
    slots = slots > kPairSlotsMax ? kPairSlotsMax : slots;
    return slots - slots % kPairProd;                       // split evenly between the producers
}

// key = (k << 16) | v' (pair_trans_kernel) and PairEntry.k are 16-bit in k: layers < 32768
bool pair_supported(int P, int nmp, int n_v, int max_L) {
    return P >= 2 && (nmp == 4 || nmp == 8) && n_v <= 65535 && max_L < 32768;
}

void launch_pair_trans(const Job *jobs, int n_jobs, int n_v_max, int l, int nmp, size_t buf_off, int fix_slab,
                       int unv_from, int max_grid, cudaStream_t s) {
    const int nvt = (n_v_max + kPairVB - 1) / kPairVB + kPairE;
    const int xb = (nvt + 3) / 4, items = xb * n_jobs;
    const int grid = max_grid > 0 && max_grid < items ? max_grid : items;
    pair_trans_kernel<<<grid, 128, 0, s>>>(jobs, l, nmp, buf_off, fix_slab, unv_from, xb, items);
}

void launch_pair_fixup(const Job *jobs, int n_jobs, int n_v_max, int l1, int nmp, int max_grid, cudaStream_t s) {
    const int xb = (n_v_max + 3) / 4, items = xb * n_jobs;
    const int grid = max_grid > 0 && max_grid < items ? max_grid : items;
    pair_fixup_kernel<<<grid, 128, 0, s>>>(jobs, l1, nmp, xb, items);
}

static int pair_round(int nsl) {
    int round = nsl / 2;
    if (const char *e = getenv("MADPIPE_PAIR_ROUND")) round = atoi(e) < nsl ? atoi(e) : nsl;
    if (round > 32) round = 32;
    return round < 1 ? 1 : round;
}

static int pair_smem(int np, int nmp, int nsl) {
    // slots of (np_max+1) rows; a thread of row 63 reads rows 63 and 64 (64 = the
    // next slot), and S reads up to nmp levels further: pad one row + nmp levels
    return (nsl * (kPairNp + 1) > 0 ? nsl * (np + 1) * nmp * 8 : 0) + (kPairNp + 2 - (np + 1)) * nmp * 8 + 2 * nmp * 8;
}

void launch_pair_step(const int2 *tdesc, int n_tiles, const void *lists, size_t buf_off, int cap, int nmp, int np,
                      int nsl, int grid, unsigned long long *prof, cudaStream_t s, int diag) {
    const int smem = pair_smem(np, nmp, nsl);
    const int stage_n = cap < kPairStage ? cap : kPairStage;
    const PairEntry *L = reinterpret_cast<const PairEntry *>(lists) + buf_off;
    switch (nmp) {
#define MP_CASE(N)                                                                                     \
    case N:                                                                                            \
        cudaFuncSetAttribute(pair_step_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);   \
        pair_step_kernel<N><<<grid, kPairThreads, smem, s>>>(tdesc, n_tiles, L, np, nsl, pair_round(nsl / kPairProd), stage_n, prof, diag); \
        break;
        MP_CASE(4) MP_CASE(8)
#undef MP_CASE
    }
}

int pair_blocks_per_sm(int nmp, int np, int nsl) {
    const int smem = pair_smem(np, nmp, nsl);
    int n = 0;
    switch (nmp) {
#define MP_OCC(N)                                                                                      \
    case N:                                                                                            \
        cudaFuncSetAttribute(pair_step_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);   \
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, pair_step_kernel<N>, kPairThreads, smem);     \
        break;
        MP_OCC(4) MP_OCC(8)
#undef MP_OCC
    }
    return n < 1 ? 1 : n;
}

}  // namespace mp
