// fp64_peak.cu -- the FP64 FMA throughput of this B200 (the `alu` roofline's peak, DESIGN.md
// §7.1): 148 x 8 CTAs x 256 threads, 8 independent DFMA chains per thread, CUDA events, best of
// 10.  Writes profiles/fp64_peak.json-shaped JSON to stdout.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/fp64_peak tools/fp64_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kIters = 8192;

__global__ void k_dfma(double a, double b, double *out)
{
    double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0 + 4, x5 = x0 + 5, x6 = x0 + 6,
           x7 = x0 + 7;
#pragma unroll 16
    for (int i = 0; i < kIters; i++) {
        x0 = __fma_rn(x0, a, b);
        x1 = __fma_rn(x1, a, b);
        x2 = __fma_rn(x2, a, b);
        x3 = __fma_rn(x3, a, b);
        x4 = __fma_rn(x4, a, b);
        x5 = __fma_rn(x5, a, b);
        x6 = __fma_rn(x6, a, b);
        x7 = __fma_rn(x7, a, b);
    }
    const double s = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
    if (s == 1.2345)
        out[0] = s;
}

int main()
{
    double *out;
    cudaMalloc(&out, 8);
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int blocks = sms * 8, tpb = 256;
    float best = 1e30f;
    for (int rep = 0; rep < 10; rep++) {
        cudaEventRecord(a);
        k_dfma<<<blocks, tpb>>>(0.999999, 1e-9, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        if (rep > 0 && ms < best)
            best = ms;
    }
    const double fmas = (double)blocks * tpb * kIters * 8;
    const double tflops = 2 * fmas / (best * 1e-3) / 1e12;
    const double lanes = fmas / (best * 1e-3) / sms / (clk * 1e3);
    printf("{\"tflops\": %.3f, \"dfma_per_s\": %.4e, \"lanes_per_sm_per_clk_at_max_clock\": %.2f, \"sms\": %d, "
           "\"clock_khz\": %d, \"ms\": %.4f, \"how\": \"%d CTAs x %d threads x %d iterations x 8 independent DFMA "
           "chains, best of 9 after a warm-up, CUDA events; tflops counts an FMA as 2 flops\"}\n",
           tflops, fmas / (best * 1e-3), lanes, sms, clk, best, blocks, tpb, kIters);
    return cudaGetLastError() != cudaSuccess;
}
