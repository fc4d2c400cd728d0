// store_probe.cu -- scattered global-store throughput on this B200 (what bounds a counting
// sort's scatter): N stores of W bytes, each lane to its own random stream.
//   random:   every store to a uniformly random W-byte slot of a B-byte array
//   frontier: S streams (cursors in a table), a store appends to a random stream, so the
//             live partial sectors are S x 32 B (a counting sort's scatter with S = CTAs x buckets)
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/store_probe tools/store_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int W>
struct Word;
template <> struct Word<4> { using T = uint32_t; };
template <> struct Word<8> { using T = uint64_t; };
template <> struct Word<16> { using T = uint4; };

// random: slot = hash(i) mod nslots
template <int W>
__global__ void k_random(typename Word<W>::T *a, uint64_t nslots, uint64_t n)
{
    using T = typename Word<W>::T;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t x = (i + 1) * 0x9E3779B97F4A7C15ull;
        x ^= x >> 29;
        x *= 0xBF58476D1CE4E5B9ull;
        x ^= x >> 32;
        T v;
        memset(&v, (int)i, sizeof(T));
        a[x % nslots] = v;
    }
}

// frontier: CTA c owns streams [c S_cta, (c + 1) S_cta); a store picks a random stream of its
// CTA and appends at the stream's shared-memory cursor (the counting sort's scatter, with
// stream s's region at s * cap)
template <int W>
__global__ void k_frontier(typename Word<W>::T *a, int s_cta, uint32_t cap, uint64_t per_cta)
{
    using T = typename Word<W>::T;
    extern __shared__ uint32_t cur[];
    for (int s = threadIdx.x; s < s_cta; s += blockDim.x)
        cur[s] = 0;
    __syncthreads();
    for (uint64_t i = threadIdx.x; i < per_cta; i += blockDim.x) {
        uint64_t x = (blockIdx.x * per_cta + i + 1) * 0x9E3779B97F4A7C15ull;
        x ^= x >> 29;
        x *= 0xBF58476D1CE4E5B9ull;
        x ^= x >> 32;
        const int s = (int)(x % (uint64_t)s_cta);
        const uint32_t k = atomicAdd(&cur[s], 1u);
        if (k < cap) {
            T v;
            memset(&v, (int)i, sizeof(T));
            a[((uint64_t)blockIdx.x * s_cta + s) * cap + k] = v;
        }
    }
}

static float time_it(void (*launch)(void *), void *arg)
{
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    launch(arg);
    cudaEventRecord(e0);
    for (int r = 0; r < 3; r++)
        launch(arg);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms / 3;
}

struct Args {
    void *a;
    uint64_t nslots, n;
    int s_cta;
    uint32_t cap;
    int ctas;
};

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const uint64_t bytes = uint64_t(4) << 30;
    void *a;
    cudaMalloc(&a, bytes);
    const uint64_t n = 100000000ull;
    static Args A;
    A.a = a;
    A.n = n;
    for (uint64_t region : {uint64_t(16) << 20, uint64_t(64) << 20, uint64_t(400) << 20}) {
        A.nslots = region / 4;
        float ms = time_it([](void *p) { Args *x = (Args *)p; k_random<4><<<148 * 8, 256>>>((uint32_t *)x->a, x->nslots, x->n); }, &A);
        printf("{\"probe\": \"random4\", \"region_MB\": %llu, \"stores\": %llu, \"ms\": %.3f, \"Gstores_s\": %.1f}\n",
               (unsigned long long)(region >> 20), (unsigned long long)n, ms, n / ms / 1e6);
        A.nslots = region / 8;
        ms = time_it([](void *p) { Args *x = (Args *)p; k_random<8><<<148 * 8, 256>>>((uint64_t *)x->a, x->nslots, x->n); }, &A);
        printf("{\"probe\": \"random8\", \"region_MB\": %llu, \"stores\": %llu, \"ms\": %.3f, \"Gstores_s\": %.1f}\n",
               (unsigned long long)(region >> 20), (unsigned long long)n, ms, n / ms / 1e6);
    }
    // frontier: 148 CTAs x S streams, 100M appends in total
    cudaFuncSetAttribute(k_frontier<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(k_frontier<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    for (int s_cta : {1024, 4096, 8192, 16384, 49152}) {
        A.ctas = sms;
        A.s_cta = s_cta;
        const uint64_t per_cta = n / sms;
        A.nslots = per_cta;
        // per-stream capacity: mean + slack, capped by the buffer
        uint64_t cap = per_cta / s_cta * 5 / 4 + 64;
        while ((uint64_t)sms * s_cta * cap * 8 > bytes)
            cap /= 2;
        A.cap = (uint32_t)cap;
        for (int w : {4, 8}) {
            float ms;
            if (w == 4)
                ms = time_it([](void *p) { Args *x = (Args *)p; k_frontier<4><<<x->ctas, 1024, x->s_cta * 4>>>((uint32_t *)x->a, x->s_cta, x->cap, x->nslots); }, &A);
            else
                ms = time_it([](void *p) { Args *x = (Args *)p; k_frontier<8><<<x->ctas, 1024, x->s_cta * 4>>>((uint64_t *)x->a, x->s_cta, x->cap, x->nslots); }, &A);
            printf("{\"probe\": \"frontier%d\", \"streams_per_cta\": %d, \"frontier_MB\": %.1f, \"cap\": %u, \"ms\": %.3f, "
                   "\"Gstores_s\": %.1f, \"err\": \"%s\"}\n",
                   w, s_cta, sms * (double)s_cta * 32 / 1048576.0, A.cap, ms, (double)per_cta * sms / ms / 1e6,
                   cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
