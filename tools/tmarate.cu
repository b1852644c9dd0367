// tmarate.cu -- how many cp.async.bulk requests per second can one B200 sustain?
//
// The step kernels stream one source-row segment per bulk copy.  This tool issues
// bulk copies with NO consumer work: each producer warp's lane 0 keeps `inflight`
// copies outstanding in its own ring of slots (it waits for the copy issued
// `inflight` requests ago, then issues the next), from random segment-aligned
// offsets of a source buffer that is either L2-resident (32 MB) or HBM-resident
// (4 GB).  Printed: requests/s and GB/s for segment size x warps/CTA x CTAs/SM.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tmarate tools/tmarate.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void tma_kernel(const char *buf, size_t nseg, uint32_t seg, int inflight, int iters,
                           unsigned long long *sink) {
    extern __shared__ __align__(128) unsigned char ring[];
    __shared__ __align__(8) uint64_t bars[8 * 32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nw = blockDim.x >> 5;
    if (threadIdx.x == 0) {
        for (int i = 0; i < nw * inflight; i++)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[i])) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (lane != 0) return;
    uint64_t x = 0x9E3779B97F4A7C15ull * (blockIdx.x * 64 + warp + 1);
    unsigned char *my = ring + (size_t)warp * inflight * seg;
    for (int i = 0; i < iters; i++) {
        const int s = i % inflight;
        const uint32_t bar = smem_u32(&bars[warp * inflight + s]);
        if (i >= inflight) {
            const uint32_t par = (uint32_t)((i / inflight - 1) & 1);
            asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
                         "@!P1 bra W;\n}\n" ::"r"(bar), "r"(par) : "memory");
        }
        x ^= x << 13; x ^= x >> 7; x ^= x << 17;
        const char *src = buf + ((x >> 16) & (nseg - 1)) * seg;   // nseg is a power of two
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(seg) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(smem_u32(my + (size_t)s * seg)), "l"(src), "r"(seg), "r"(bar) : "memory");
    }
    for (int s = 0; s < inflight && s < iters; s++) {   // drain
        const int i = iters - 1 - s;
        const uint32_t bar = smem_u32(&bars[warp * inflight + (i % inflight)]);
        const uint32_t par = (uint32_t)((i / inflight) & 1);
        asm volatile("{\n.reg .pred P1;\nW2:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
                     "@!P1 bra W2;\n}\n" ::"r"(bar), "r"(par) : "memory");
    }
    if (warp == 0) atomicAdd(sink, (unsigned long long)my[0]);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t big = 4ull << 30, small = 32ull << 20;
    char *buf;
    cudaMalloc(&buf, big);
    cudaMemset(buf, 1, big);
    unsigned long long *sink;
    cudaMalloc(&sink, 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const uint32_t segs[] = {1024, 4096};
    const int warps_l[] = {1, 2, 4, 8};
    const int ctas_l[] = {1, 2};
    for (int res = 1; res < 2; res++)
        for (uint32_t seg : segs)
            for (int ctas : ctas_l)
                for (int warps : warps_l) {
                    const size_t bytes = res ? big : small;
                    int inflight = (int)((96 * 1024) / ((size_t)warps * seg));
                    if (inflight > 32) inflight = 32;
                    if (inflight < 2) continue;
                    const int smem = warps * inflight * seg;
                    cudaFuncSetAttribute(tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                    const int iters = 4000;
                    const int grid = sms * ctas;
                    tma_kernel<<<grid, 32 * warps, smem>>>(buf, bytes / seg, seg, inflight, 200, sink);
                    cudaEventRecord(a);
                    tma_kernel<<<grid, 32 * warps, smem>>>(buf, bytes / seg, seg, inflight, iters, sink);
                    cudaEventRecord(b);
                    cudaEventSynchronize(b);
                    float ms = 0.f;
                    cudaEventElapsedTime(&ms, a, b);
                    const double req = (double)grid * warps * iters;
                    printf("{\"src\": \"%s\", \"seg\": %u, \"ctas_per_sm\": %d, \"warps\": %d, \"inflight_per_warp\": %d, "
                           "\"Greq_s\": %.3f, \"GBps\": %.1f, \"err\": \"%s\"}\n",
                           res ? "hbm" : "l2", seg, ctas, warps, inflight, req / (ms * 1e-3) / 1e9,
                           req * seg / (ms * 1e-3) / 1e9, cudaGetErrorString(cudaGetLastError()));
                    fflush(stdout);
                }
    return 0;
}
