// mp_step_tma.cu -- the wavefront min-plus step (a3-a5) as a TMA-pipelined,
// warp-specialised sm_100a kernel.
//
// Same recursion as step_kernel in mp_kernels.cu (decision form Q1):
//   A[l][v][p][m] = clamp_tau( min over live k of
//        N: A[k-1][v'][p-1][m]            (normal GPU fits)
//        S: U(k,l) + A[k-1][v'][p][m+d]   (special GPU) )
// What changes is how the source rows reach the SM:
//   * a CTA owns VB delay rows x np processor rows of one job (one (l, v) row
//     group per warp-aligned slice, so every warp sees ONE transition per k and
//     the shift d is warp-uniform);
//   * the live transitions (k, v) of the CTA are computed once into shared
//     memory (a3), the k with at least one live row are compacted;
//   * a producer warp streams, for each such k, the needed source row segments
//     A[k-1][v'][p_lo-1 .. p_lo+np-1][*] into an NST-stage shared-memory ring
//     with cp.async.bulk (TMA bulk copies) completing on an mbarrier;
//   * consumer threads each own a (p, m-pair) of one row: N is one 16-byte
//     shared load, S one 16-byte load (d even) or two 8-byte loads (d odd),
//     then a DADD and two min's per level; the clamp is fused into the store.
// No result depends on the order in which k are combined (min is exact).
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

constexpr int kNst = 6;              // pipeline stages
constexpr int kConsumers = 256;      // consumer threads (8 warps) + 1 producer warp
constexpr int kTmaTrans = 2048;      // staged transition entries per chunk
constexpr int kTmaKChunk = 512;

template <int NMP>
__global__ void __launch_bounds__(kConsumers + 32, 3) step_tma_kernel(const Job *__restrict__ jobs,
                                                                   const int32_t *__restrict__ tile_job,
                                                                   int l) {
    constexpr int HP = NMP / 2;          // m-pairs per processor row
    extern __shared__ __align__(128) unsigned char dsm[];
    __shared__ Job sJ;
    __shared__ __align__(8) uint64_t full[kNst];
    __shared__ __align__(8) uint64_t empty[kNst];
    __shared__ int32_t s_tr[kTmaTrans];
    __shared__ double s_U[kTmaKChunk];
    __shared__ int16_t s_act[kTmaKChunk];
    __shared__ int s_nact;

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const int jid = tile_job[blockIdx.x];
    if (tid == 0) {
        sJ = jobs[jid];
        for (int s = 0; s < kNst; s++) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumers / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
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

    // base row p = 0 (reading Q10)
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

    // consumer geometry: row group = np*HP threads padded to whole warps
    const int rowgroup = ((np * HP + 31) / 32) * 32;
    const int vv = tid / rowgroup;
    const int q = tid - vv * rowgroup;
    const int pp_off = q / HP;
    const int h = q - pp_off * HP;
    const bool consumer = warp < kConsumers / 32;
    const bool active = consumer && vv < vcount && pp_off < np;
    const int seg_doubles = (np + 1) * NMP;                 // rows p_lo-1 .. p_lo+np-1
    const uint32_t seg_bytes = (uint32_t)seg_doubles * 8u;
    double *ring = reinterpret_cast<double *>(dsm);          // [kNst][vb][seg_doubles]
    const int vb = J.vb;

    double best0 = MP_INF, best1 = MP_INF;
    const int kmin = max(kmin_of(J, l), kmin_mem(J, l));
    const int kc_len = min(kTmaKChunk, kTmaTrans / vcount);
    const double *__restrict__ tab = J.table;
    int gi = 0;   // running pipeline index (phases continue across chunks)

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
        if (pt == 0) {   // each live (k, l, v) feeds (P-1) n_m relaxations
            for (int o = 16; o > 0; o >>= 1) live += __shfl_xor_sync(0xffffffffu, live, o);
            if (lane == 0 && live)
                atomicAdd(J.eff, (unsigned long long)live * (unsigned long long)(J.P - 1) *
                                     (unsigned long long)n_m);
        }
        __syncthreads();
        if (warp == 0) {   // compact the k that have at least one live row
            int base = 0;
            for (int kb = 0; kb < nk; kb += 32) {
                const int kk = kb + lane;
                bool any = false;
                if (kk < nk)
                    for (int v2 = 0; v2 < vcount; v2++) any |= s_tr[kk * vcount + v2] >= 0;
                const unsigned bal = __ballot_sync(0xffffffffu, any);
                if (any) s_act[base + __popc(bal & ((1u << lane) - 1u))] = (int16_t)kk;
                base += __popc(bal);
            }
            if (lane == 0) s_nact = base;
        }
        __syncthreads();
        const int nact = s_nact;
        if (!consumer) {
            // ---------------- producer warp: one elected lane issues the bulk copies
            if (lane == 0) {
                for (int i = 0; i < nact; i++, gi++) {
                    const int s = gi % kNst;
                    if (gi >= kNst) mbar_wait(&empty[s], (uint32_t)((gi / kNst - 1) & 1));
                    const int kk = s_act[i];
                    const int k = kc0 + kk;
                    uint32_t bytes = 0;
                    for (int v2 = 0; v2 < vcount; v2++) bytes += s_tr[kk * vcount + v2] >= 0 ? seg_bytes : 0u;
                    mbar_arrive_expect_tx(&full[s], bytes);
                    const double *src_slab = tab + (size_t)(k - 1) * slab + (size_t)(p_lo - 1) * NMP;
                    for (int v2 = 0; v2 < vcount; v2++) {
                        const int32_t tr = s_tr[kk * vcount + v2];
                        if (tr < 0) continue;
                        const int vn = tr & 0xFFFF;
                        bulk_g2s(ring + ((size_t)s * vb + v2) * seg_doubles, src_slab + (size_t)vn * rowlen,
                                 seg_bytes, &full[s]);
                    }
                }
            } else {
                gi += nact;
            }
        } else {
            // ---------------- consumers
            for (int i = 0; i < nact; i++, gi++) {
                const int s = gi % kNst;
                mbar_wait(&full[s], (uint32_t)((gi / kNst) & 1));
                const int kk = s_act[i];
                const int32_t tr = active ? s_tr[kk * vcount + vv] : -1;
                if (tr >= 0) {
                    const double *seg = ring + ((size_t)s * vb + vv) * seg_doubles;
                    if (tr & (1 << 24)) {     // N: row p-1 of the segment (offset pp_off)
                        const double2 x = *reinterpret_cast<const double2 *>(seg + pp_off * NMP + 2 * h);
                        best0 = x.x < best0 ? x.x : best0;
                        best1 = x.y < best1 ? x.y : best1;
                    }
                    const int d = (tr >> 16) & 0xFF;
                    const int m0 = 2 * h + d;
                    if (m0 <= n_m - 1) {      // S: row p (offset pp_off+1), levels m0, m0+1
                        const double U = s_U[kk];
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
                __syncwarp();
                if (lane == 0) mbar_arrive(&empty[s]);
            }
        }
    }
    if (active) {
        double2 r;
        r.x = (2 * h < n_m && best0 <= tau) ? best0 : MP_INF;
        r.y = (2 * h + 1 < n_m && best1 <= tau) ? best1 : MP_INF;
        *reinterpret_cast<double2 *>(out + (size_t)(v0 + vv) * rowlen + (size_t)(p_lo + pp_off) * NMP + 2 * h) = r;
    }
}

int tma_smem_bytes(int vb, int np, int nmp) { return kNst * vb * (np + 1) * nmp * 8; }

// geometry of the TMA step kernel for one job: np processor rows (np*nmp/2
// threads, padded to whole warps) x vb delay rows per CTA
void tma_geom(int P, int n_v, int nmp, int *vb, int *np, int *n_ptiles, int *n_tiles) {
    const int rows = P - 1 > 0 ? P - 1 : 1;
    const int hp = nmp / 2;
    int cap = kConsumers / hp;             // processor rows that fit in 256 threads
    if (cap < 1) cap = 1;
    *np = rows < cap ? rows : cap;
    *n_ptiles = (rows + *np - 1) / *np;
    const int rowgroup = ((*np * hp + 31) / 32) * 32;
    int v = kConsumers / rowgroup;
    if (v < 1) v = 1;
    if (v > n_v) v = n_v;
    *vb = v;
    *n_tiles = ((n_v + *vb - 1) / *vb) * *n_ptiles;
}

void launch_step_tma(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp, int smem,
                     cudaStream_t s) {
    switch (nmp) {
#define MP_CASE(N)                                                                                  \
    case N:                                                                                         \
        cudaFuncSetAttribute(step_tma_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); \
        step_tma_kernel<N><<<n_tiles, kConsumers + 32, smem, s>>>(jobs, tile_job, l);              \
        break;
        MP_CASE(2) MP_CASE(4) MP_CASE(8) MP_CASE(16) MP_CASE(32) MP_CASE(64)
#undef MP_CASE
    }
}

}  // namespace mp
