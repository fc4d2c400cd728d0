// atoms_probe.cu -- shared-memory atomic throughput on this B200 (the sort's histogram and
// ranking primitives): cycles per warp instruction for random addresses over W words,
//   red      atomicAdd(&s[a], 1) with the result unused (ATOMS.POPC.INC RZ)
//   ret      atomicAdd(&s[a], 1) with the result used   (ATOMS.POPC.INC Rd)
//   retv     atomicAdd(&s[a], v) with the result used   (ATOMS.ADD Rd)
//   rmw      s[a] = s[a] + 1 (plain LDS + STS, racy: a cost reference only)
//   match    __match_any_sync on the address + one lane's ATOMS.ADD per group
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/atoms_probe tools/atoms_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kTpb = 1024, kIters = 4096;

template <int MODE>
__global__ void __launch_bounds__(kTpb) k_probe(int words, unsigned *sink)
{
    extern __shared__ unsigned s[];
    for (int i = threadIdx.x; i < words; i += kTpb)
        s[i] = 0;
    __syncthreads();
    uint32_t x = 0x9E3779B9u * (blockIdx.x * kTpb + threadIdx.x + 1);
    unsigned acc = 0;
    const uint32_t mask = (uint32_t)words - 1; // words: a power of two
#pragma unroll 8
    for (int it = 0; it < kIters; it++) {
        x = x * 1664525u + 1013904223u;
        uint32_t h = x ^ (x >> 16); // per-lane hash: the LCG alone is affine in the lane
        h *= 0x85EBCA6Bu;           // (conflict-free arithmetic progressions of addresses)
        h ^= h >> 13;
        h *= 0xC2B2AE35u;
        h ^= h >> 16;
        const uint32_t a = h & mask;
        if (MODE == 0) {
            atomicAdd(&s[a], 1u);
        } else if (MODE == 1) {
            acc += atomicAdd(&s[a], 1u);
        } else if (MODE == 2) {
            acc += atomicAdd(&s[a], (x & 7u) + 1u);
        } else if (MODE == 5) {
            acc += a;
        } else if (MODE == 3) {
            volatile unsigned *vs = s;
            vs[a] = vs[a] + 1u;
        } else {
            const unsigned g = __match_any_sync(0xffffffffu, a);
            const int leader = __ffs(g) - 1;
            const int lane = threadIdx.x & 31;
            unsigned base = 0;
            if (lane == leader)
                base = atomicAdd(&s[a], (unsigned)__popc(g));
            base = __shfl_sync(0xffffffffu, base, leader);
            acc += base + __popc(g & ((1u << lane) - 1u));
        }
    }
    __syncthreads();
    if (acc == 0x12345678u)
        sink[0] = acc;
    if (threadIdx.x == 0)
        atomicAdd(sink + 1, s[0]);
}

template <int MODE> static void run(const char *name, int words, int sms, unsigned *sink)
{
    const int smem = words * 4;
    cudaFuncSetAttribute(k_probe<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_probe<MODE>, kTpb, smem);
    const int blocks = sms * (per_sm > 0 ? per_sm : 1);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    k_probe<MODE><<<blocks, kTpb, smem>>>(words, sink);
    cudaEventRecord(a);
    const int reps = 5;
    for (int r = 0; r < reps; r++)
        k_probe<MODE><<<blocks, kTpb, smem>>>(words, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const double warp_ops = (double)reps * blocks * (kTpb / 32) * kIters;
    const double sm_cycles = ms * 1e-3 * clk_khz * 1e3; // per SM
    printf("{\"probe\": \"%s\", \"words\": %d, \"ctas_per_sm\": %d, \"ms\": %.3f, \"cycles_per_warp_op\": %.2f, "
           "\"cycles_per_lane\": %.3f, \"err\": \"%s\"}\n",
           name, words, per_sm, ms / reps, sm_cycles * sms / warp_ops, sm_cycles * sms / warp_ops / 32,
           cudaGetErrorString(cudaGetLastError()));
}

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned *sink;
    cudaMalloc(&sink, 16);
    for (int words : {1024, 4096, 32768}) {
        run<5>("hashonly", words, sms, sink);
        run<0>("red", words, sms, sink);
        run<1>("ret", words, sms, sink);
        run<2>("retv", words, sms, sink);
        run<3>("rmw", words, sms, sink);
        run<4>("match", words, sms, sink);
    }
    return 0;
}
