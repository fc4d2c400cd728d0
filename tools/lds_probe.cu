// lds_probe.cu -- shared-memory load throughput on this B200 for the access patterns of the
// staged lookup kernel: how many L1/shared data-pipe cycles does a warp-wide
// 16 B / 8 B load cost when its 32 lanes read 1, 2, 4, ... distinct interval records (112 B
// apart)?  Throughput test: 148 x 8 CTAs x 256 threads, each thread 4096 loads, CUDA events.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/lds_probe tools/lds_probe.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kRecDoubles = 14; // 112 B interval record
constexpr int kRecs = 64;
constexpr int kIters = 4096;

// record index of lane `lane` for pattern p
__device__ __forceinline__ int rec_of(int p, int lane)
{
    switch (p) {
    case 0: return 0;                    // all lanes one record (broadcast)
    case 1: return lane >> 4;            // 2 records, half-warps
    case 2: return lane & 1;             // 2 records, alternating lanes
    case 3: return lane >> 3;            // 4 records, quarter-warps
    case 4: return lane >= 28 ? 1 : 0;   // 2 records, 4 lanes on the second
    case 5: return lane >> 2;            // 8 records
    case 6: return lane;                 // 32 records
    case 7: return (lane >> 4) * 8;      // 2 records 8 apart (same banks: 8 x 28 = 224 = 0 mod 32)
    default: return 0;
    }
}

template <int BYTES>
__global__ void k_probe(int p, double *out)
{
    __shared__ __align__(16) double rec[kRecs * kRecDoubles];
    for (int i = threadIdx.x; i < kRecs * kRecDoubles; i += blockDim.x)
        rec[i] = i * 0.5;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int r = rec_of(p, lane);
    const double *base = rec + r * kRecDoubles;
    unsigned acc = 0;
    const unsigned a0 = (unsigned)__cvta_generic_to_shared(base);
#pragma unroll 1
    for (int it = 0; it < kIters / 7; it++) {
#pragma unroll
        for (int f = 0; f < 7; f++) { // 7 independent loads per trip (the fields of a record)
            const unsigned addr = a0 + f * 16;
            if constexpr (BYTES == 16) {
                unsigned x, y, z, w;
                asm volatile("ld.volatile.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                             : "=r"(x), "=r"(y), "=r"(z), "=r"(w) : "r"(addr));
                acc ^= x ^ y ^ z ^ w;
            } else if constexpr (BYTES == 8) {
                unsigned x, y;
                asm volatile("ld.volatile.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(addr));
                acc ^= x ^ y;
            } else {
                unsigned x;
                asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(x) : "r"(addr));
                acc ^= x;
            }
        }
    }
    if (acc == 12345678u)
        out[0] = (double)acc;
}

int main()
{
    double *out;
    cudaMalloc(&out, 8);
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const char *names[] = {"1 record", "2 records (half-warps)", "2 records (alternating)", "4 records",
                           "2 records (4 lanes)", "8 records", "32 records", "2 records, same banks"};
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    printf("{\"sms\": %d, \"clock_khz\": %d, \"iters\": %d, \"results\": [\n", sms, clk, kIters);
    bool first = true;
    for (int bytes : {16, 8, 4})
        for (int p = 0; p < 8; p++) {
            float best = 1e30f;
            for (int rep = 0; rep < 5; rep++) {
                cudaEventRecord(a);
                if (bytes == 16)
                    k_probe<16><<<sms * 8, 256>>>(p, out);
                else if (bytes == 8)
                    k_probe<8><<<sms * 8, 256>>>(p, out);
                else
                    k_probe<4><<<sms * 8, 256>>>(p, out);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                float ms = 0;
                cudaEventElapsedTime(&ms, a, b);
                if (ms < best)
                    best = ms;
            }
            const double warp_loads = (double)sms * 8 * 8 * (kIters / 7) * 7; // warps x loads
            const double per_sm_clk = warp_loads / sms / (best * 1e-3 * clk * 1e3);
            printf("%s {\"bytes\": %d, \"pattern\": \"%s\", \"ms\": %.4f, \"warp_loads_per_sm_per_clk\": %.4f, "
                   "\"clk_per_warp_load\": %.3f}",
                   first ? "" : ",\n", bytes, names[p], best, per_sm_clk, 1.0 / per_sm_clk);
            first = false;
        }
    printf("\n]}\n");
    return cudaGetLastError() != cudaSuccess;
}
