// racecheck_repro.cu -- minimal repro of the racecheck reports on the persistent step
// kernels (profiles/r02_sanitize_*.md): compute-sanitizer racecheck flags shared-memory
// handoffs that are ordered only by an mbarrier (and by TMA completion on it), i.e. the
// producer/consumer protocol of step_persist_kernel and pair_step_kernel.
//
// One CTA, two warps, a 2-slot ring of 1 KB slots, 64 rounds.  Warp 1 (producer) fills a
// slot -- either with generic shared stores (MODE 0, then mbarrier.arrive, which has
// release semantics) or with a cp.async.bulk global->shared copy completing on the slot's
// full barrier (MODE 1, the kernels' pattern) -- and warp 0 (consumer) waits on the full
// barrier (try_wait: acquire), reads the slot, then arrives on the slot's empty barrier,
// which the producer waits on before refilling the slot.  Under the PTX memory model
// every read is ordered after the write it reads and before the next write to the slot;
// the kernel checks the values it reads (mismatches -> bad != 0).  Racecheck nevertheless
// reports RAW / WAR hazards between the two warps on every slot.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o tools/racecheck_repro tools/racecheck_repro.cu
//   compute-sanitizer --tool racecheck tools/racecheck_repro
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint32_t b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(n) : "memory");
}
__device__ __forceinline__ void mb_arrive(uint32_t b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory");
}
__device__ __forceinline__ void mb_expect(uint32_t b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mb_wait(uint32_t b, uint32_t par) {
    asm volatile("{\n.reg .pred P1;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W_%=;\n}\n" ::"r"(b),
                 "r"(par) : "memory");
}

template <int MODE>
__global__ void ring(const double *src, int rounds, int *bad) {
    constexpr int SLOT = 128;                      // doubles per slot (1 KB)
    __shared__ __align__(128) double slot[2][SLOT];
    __shared__ __align__(8) uint64_t full[2], empty[2];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < 2; s++) { mb_init(sa(&full[s]), 1); mb_init(sa(&empty[s]), 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    int errs = 0;
    for (int r = 0; r < rounds; r++) {
        const int s = r & 1, use = r >> 1;
        if (warp == 1) {                                                   // producer
            if (use > 0) mb_wait(sa(&empty[s]), (use - 1) & 1);
            if (MODE == 0) {
                for (int i = lane; i < SLOT; i += 32) slot[s][i] = (double)(r * SLOT + i);
                __syncwarp();
                if (lane == 0) mb_arrive(sa(&full[s]));
            } else if (lane == 0) {
                mb_expect(sa(&full[s]), SLOT * 8);
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                                 sa(&slot[s][0])),
                             "l"(src + (size_t)r * SLOT), "r"(SLOT * 8), "r"(sa(&full[s]))
                             : "memory");
            }
        } else {                                                           // consumer
            mb_wait(sa(&full[s]), use & 1);
            for (int i = lane; i < SLOT; i += 32) errs += slot[s][i] != (double)(r * SLOT + i);
            __syncwarp();
            if (lane == 0) mb_arrive(sa(&empty[s]));
        }
    }
    if (errs) atomicAdd(bad, errs);
}

int main() {
    const int rounds = 64;
    double *src;
    int *bad;
    cudaMalloc(&src, sizeof(double) * 128 * rounds);
    cudaMallocManaged(&bad, sizeof(int));
    double *h = new double[128 * rounds];
    for (int i = 0; i < 128 * rounds; i++) h[i] = (double)i;
    cudaMemcpy(src, h, sizeof(double) * 128 * rounds, cudaMemcpyHostToDevice);
    *bad = 0;
    ring<0><<<1, 64>>>(src, rounds, bad);
    cudaDeviceSynchronize();
    const int b0 = *bad;
    *bad = 0;
    ring<1><<<1, 64>>>(src, rounds, bad);
    cudaError_t e = cudaDeviceSynchronize();
    printf("{\"generic_store_mismatches\": %d, \"bulk_copy_mismatches\": %d, \"cuda\": \"%s\"}\n", b0, *bad,
           cudaGetErrorString(e));
    return 0;
}
