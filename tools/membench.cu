// membench.cu -- what HBM bandwidth can the step kernel's access pattern reach?
//
// The persistent step kernel streams source-row segments of S bytes (4 KB at the
// GPT config) from random rows of multi-GB DP tables into shared memory with
// cp.async.bulk, a few dozen in flight per SM.  This tool measures exactly that
// pattern with no DP work: 2 CTAs per SM, one producer warp issuing bulk copies
// of random S-byte segments into an NST-slot ring, 8 consumer warps that only
// wait for each slot and release it.  It prints GB/s per segment size, plus a
// plain sequential device-to-device copy for reference.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/membench tools/membench.cu
//   ./tools/membench
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(288, 2) ring_kernel(const char *buf, const uint64_t *offs, int n_per_cta,
                                                      uint32_t seg, int nst, double *sink) {
    extern __shared__ __align__(128) unsigned char ring[];
    __shared__ __align__(8) uint64_t full[32], empty[32];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) {
        for (int s = 0; s < nst; s++) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&full[s])), "r"(1));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&empty[s])), "r"(8));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const uint64_t *my = offs + (size_t)blockIdx.x * n_per_cta;
    if (warp == 8) {
        for (int i0 = 0; i0 < n_per_cta; i0 += nst) {
            const int i = i0 + lane;
            if (lane < nst && i < n_per_cta) {
                const int s = lane, use = i0 / nst;
                if (use > 0) {
                    asm volatile("{\n.reg .pred P1;\nW1:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
                                 "@!P1 bra W1;\n}\n" ::"r"(smem_u32(&empty[s])), "r"((use - 1) & 1) : "memory");
                }
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(smem_u32(ring + (size_t)s * seg)), "l"(buf + my[i]), "r"(seg),
                             "r"(smem_u32(&full[s])) : "memory");
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[s])),
                             "r"(seg) : "memory");
            }
            __syncwarp();
        }
        return;
    }
    double acc = 0.0;
    for (int i = 0; i < n_per_cta; i++) {
        const int s = i % nst, ph = (i / nst) & 1;
        asm volatile("{\n.reg .pred P1;\nW2:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
                     "@!P1 bra W2;\n}\n" ::"r"(smem_u32(&full[s])), "r"(ph) : "memory");
        acc += reinterpret_cast<const double *>(ring + (size_t)s * seg)[tid & 7];
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[s])) : "memory");
    }
    if (acc == 12345.678) *sink = acc;
}

int main() {
    const size_t bytes = (size_t)16 << 30;   // 16 GB of "tables"
    char *buf;
    if (cudaMalloc(&buf, bytes) != cudaSuccess) { printf("alloc failed\n"); return 1; }
    cudaMemset(buf, 0, bytes);
    double *sink;
    cudaMalloc(&sink, 8);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int ctas = 2 * sms;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    // reference: sequential copy
    {
        char *dst;
        cudaMalloc(&dst, (size_t)4 << 30);
        for (int r = 0; r < 3; r++) cudaMemcpy(dst, buf, (size_t)4 << 30, cudaMemcpyDeviceToDevice);
        cudaEventRecord(a);
        for (int r = 0; r < 5; r++) cudaMemcpy(dst, buf, (size_t)4 << 30, cudaMemcpyDeviceToDevice);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("{\"pattern\": \"cudaMemcpy D2D 4 GiB (read+write)\", \"GBps\": %.1f}\n",
               5.0 * 2.0 * (double)((size_t)4 << 30) / (ms / 1e3) / 1e9);
        cudaFree(dst);
    }
    for (uint32_t seg : {1024u, 2048u, 4096u, 8192u, 16384u}) {
        for (int ring_kb : {96}) {
            const int nst = std::min(32, (int)((ring_kb * 1024) / seg));
            const int n_per_cta = 4096;
            std::vector<uint64_t> h((size_t)ctas * n_per_cta);
            uint64_t x = 88172645463325252ull;
            const uint64_t nseg = bytes / seg;
            for (auto &o : h) {
                x ^= x << 13; x ^= x >> 7; x ^= x << 17;
                o = (x % nseg) * seg;
            }
            uint64_t *offs;
            cudaMalloc(&offs, h.size() * 8);
            cudaMemcpy(offs, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
            const int smem = nst * seg;
            cudaFuncSetAttribute(ring_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            for (int r = 0; r < 2; r++) ring_kernel<<<ctas, 288, smem>>>(buf, offs, n_per_cta, seg, nst, sink);
            cudaEventRecord(a);
            const int reps = 5;
            for (int r = 0; r < reps; r++) ring_kernel<<<ctas, 288, smem>>>(buf, offs, n_per_cta, seg, nst, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            const cudaError_t e = cudaGetLastError();
            printf("{\"pattern\": \"cp.async.bulk random segments\", \"seg_bytes\": %u, \"nst\": %d, "
                   "\"ctas\": %d, \"GBps\": %.1f, \"err\": \"%s\"}\n",
                   seg, nst, ctas, (double)reps * h.size() * seg / (ms / 1e3) / 1e9, cudaGetErrorString(e));
            cudaFree(offs);
        }
    }
    return 0;
}
