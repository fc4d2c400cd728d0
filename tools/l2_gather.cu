// l2_gather.cu -- SURVEY.md §8d's gather microbenchmark: random 96 B record gathers (six 16 B
// loads, the pair gather of one (lookup, nuclide)) over buffers the size of the small grid's
// point records (37 MB: L2-resident), the large grid's (193 MB) and XL's (4.07 GB), plus the
// L2 attributes §8d asks to query.  Prints one JSON object.  Development/measurement tool.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2_gather tools/l2_gather.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t x)
{
    x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
    return x;
}

template <int ILP>
__global__ void __launch_bounds__(256) k_gather(const double2 *__restrict__ buf, uint64_t nrec, int iters,
                                                 double *__restrict__ sink)
{
    const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    double acc = 0.0;
    for (int it = 0; it < iters; it++) {
        double2 v[ILP][6];
#pragma unroll
        for (int u = 0; u < ILP; u++) {
            const uint64_t rec = mix(tid * 1315423911ull + (uint64_t)(it * ILP + u) * 2654435761ull) % nrec;
            const double2 *p = buf + rec * 6;
#pragma unroll
            for (int k = 0; k < 6; k++)
                v[u][k] = __ldg(p + k);
        }
#pragma unroll
        for (int u = 0; u < ILP; u++)
#pragma unroll
            for (int k = 0; k < 6; k++)
                acc += v[u][k].x + v[u][k].y;
    }
    if (acc == 1234.5678)
        sink[0] = acc;
}

int main()
{
    int dev = 0, l2 = 0, persist = 0, window = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    cudaDeviceGetAttribute(&persist, cudaDevAttrMaxPersistingL2CacheSize, dev);
    cudaDeviceGetAttribute(&window, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const size_t sizes[3] = {size_t(36893) << 10, size_t(192603) << 10, size_t(4070) << 20};
    const char *names[3] = {"small_points_37MB", "large_points_193MB", "xl_points_4.07GB"};
    double *sink;
    cudaMalloc(&sink, 8);
    printf("{\"l2_cache_bytes\": %d, \"max_persisting_l2_bytes\": %d, \"max_access_policy_window_bytes\": %d, "
           "\"sms\": %d, \"record_bytes\": 96, \"gathers\": {", l2, persist, window, sms);
    for (int s = 0; s < 3; s++) {
        double2 *buf = nullptr;
        if (cudaMalloc(&buf, sizes[s]) != cudaSuccess) {
            printf("%s\"%s\": null", s ? ", " : "", names[s]);
            continue;
        }
        cudaMemset(buf, 0, sizes[s]);
        const uint64_t nrec = sizes[s] / 96;
        const int blocks = sms * 8, iters = 64;
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        for (int w = 0; w < 3; w++)
            k_gather<4><<<blocks, 256>>>(buf, nrec, iters, sink);
        float best = 1e30f;
        for (int r = 0; r < 10; r++) {
            cudaEventRecord(a);
            k_gather<4><<<blocks, 256>>>(buf, nrec, iters, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms = 0;
            cudaEventElapsedTime(&ms, a, b);
            best = ms < best ? ms : best;
        }
        const double bytes = (double)blocks * 256 * iters * 4 * 96;
        printf("%s\"%s\": {\"GBps_useful\": %.1f, \"records_per_s\": %.4g, \"ms\": %.4f}", s ? ", " : "", names[s],
               bytes / (best * 1e-3) / 1e9, bytes / 96 / (best * 1e-3), best);
        cudaFree(buf);
    }
    printf("}, \"how\": \"random 96 B records (6 x 16 B __ldg each, 4 independent records in flight per thread), %d CTAs x 256 threads, best of 10, CUDA events\"}\n",
           sms * 8);
    return 0;
}
