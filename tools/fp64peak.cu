// fp64peak.cu -- measured FP64-pipe throughput of this B200 for the roofline of the DP
// step kernel (BASELINE north_star: "FP64/INT pipe utilisation against peak").
//
// Three loops, each with 8 independent dependency chains per thread and enough warps
// to saturate every SM (148 SMs x 32 warps):
//   dadd : x = x + c                       (DADD, the S candidate of a relaxation)
//   dfma : x = x * a + c                   (DFMA, the datasheet's FP64 FLOP/s)
//   relax: b = (c + y < b) ? c + y : b     (DADD + DSETP + 2 FSEL: one S relaxation of
//                                           pair_step_kernel's consumer loop)
// Each prints instructions/s (per the dominant FP64 op) as one JSON line.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/fp64peak tools/fp64peak.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void loop(double *out, double a, double c, int iters) {
    double x[8];
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = threadIdx.x * 1e-3 + i;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < 8; i++) {
            if (MODE == 0) x[i] = __dadd_rn(x[i], c);
            else if (MODE == 1) x[i] = fma(x[i], a, c);
            else {
                const double cand = __dadd_rn(c, (double)i * a);
                x[i] = cand < x[i] ? cand : x[i] - a;    // keeps the chain live
            }
        }
    }
    double s = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) s += x[i];
    if (s == 12345.678) out[0] = s;
}

template <int MODE>
double rate(int sms) {
    double *out;
    cudaMalloc(&out, 8);
    const int threads = 256, blocks = sms * 8, iters = 4096;
    loop<MODE><<<blocks, threads>>>(out, 1.0000001, 1e-9, 16);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    loop<MODE><<<blocks, threads>>>(out, 1.0000001, 1e-9, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    cudaFree(out);
    return (double)blocks * threads * iters * 8 / (ms * 1e-3);
}

int main() {
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const double dadd = rate<0>(sms), dfma = rate<1>(sms), relax = rate<2>(sms);
    printf("{\"sms\": %d, \"clock_khz\": %d, \"dadd_per_s\": %.4g, \"dfma_per_s\": %.4g, \"dfma_flops\": %.4g, "
           "\"relax_per_s\": %.4g, \"dadd_lanes_per_sm_per_clk\": %.2f, "
           "\"note\": \"tools/fp64peak.cu: 8 independent chains per thread, %d CTAs x 256 threads; relax = one S "
           "relaxation (DADD + DSETP + select)\"}\n",
           sms, clk, dadd, dfma, 2 * dfma, relax, dadd / (sms * clk * 1e3), sms * 8);
    return 0;
}
