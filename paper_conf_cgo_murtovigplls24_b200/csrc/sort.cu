// sort.cu -- sampling + the (material, energy) counting sort.
//
// Key = kbase[material] + energy bucket (BucketPlan: material m gets nb[m] buckets in
// proportion to P(m) * num_nucs[m], its expected share of the pairs), K <= 49152.
//   k_bucket_count   sample each lookup of the chunk once (one Listing-7 jump per thread,
//                    then one affine step per lookup), write its energy and key at its own
//                    offset (coalesced) and histogram the keys in shared memory
//   k_bucket_colscan per bucket, exclusive scan over CTAs (loads batched by 8)
//   k_bucket_base    exclusive scan of the bucket totals + material bases (one CTA)
//   k_bucket_scatter scatter the 4 B lookup offsets to their slots: 68 MB for 17M lookups,
//                    L2-resident, so the random partial-sector writes merge in L2
//   k_bucket_gather  (split path only) q in slot order; the fused lookup kernel instead
//                    prefetches q_of[slot] one grid-stride iteration ahead
// Order inside a bucket is whatever the shared-memory atomics give; results never depend
// on it (every lookup is independent and the hash is an integer sum).
#include <algorithm>

#include "lookup_common.cuh"

namespace xs {

constexpr int kSortTpb = 1024;

__global__ void __launch_bounds__(kSortTpb) k_bucket_count(SampleView sv, BucketPlan bp, int per_cta, Affine J_tpb,
                                                            uint32_t *__restrict__ hist, double *__restrict__ q_of,
                                                            uint16_t *__restrict__ key_of)
{
    extern __shared__ uint32_t sh[];
    __shared__ int s_nb[kMaterials], s_kbase[kMaterials];
    const int K = bp.K;
    for (int k = threadIdx.x; k < K; k += kSortTpb)
        sh[k] = 0;
    if (threadIdx.x == 0) {
#pragma unroll
        for (int m = 0; m < kMaterials; m++) {
            s_nb[m] = bp.nb[m];
            s_kbase[m] = bp.kbase[m];
        }
    }
    __syncthreads();
    const int count = (int)sv.count;
    const int beg = blockIdx.x * per_cta;
    const int end = min(beg + per_cta, count);
    int j = beg + threadIdx.x;
    if (j < end) {
        uint64_t s = lookup_state(sv, j);
        for (; j < end; j += kSortTpb) {
            double q;
            int mat;
            sample_lookup(s, sv, q, mat);
            const int key = bucket_key(s_nb, s_kbase, mat, q);
            atomicAdd(&sh[key], 1u);
            q_of[j] = q;
            key_of[j] = (uint16_t)key;
            s = lcg_apply(J_tpb, s);
        }
    }
    __syncthreads();
    uint32_t *h = hist + (int64_t)blockIdx.x * K;
    for (int k = threadIdx.x; k < K; k += kSortTpb)
        h[k] = sh[k];
}

// per bucket k: exclusive scan over the CTAs, in place; total[k] = the bucket's size.
// A CTA owns 32 buckets (lane = bucket, one coalesced 128 B row segment per load) and its 8
// warps own 1/8 of the CTA rows each, so every lane keeps ~19 independent loads in flight;
// the 8 warp partials per bucket are scanned through shared memory.
constexpr int kColWarps = 8;

__global__ void __launch_bounds__(32 * kColWarps) k_bucket_colscan(int K, int ctas, uint32_t *hist,
                                                                    uint32_t *__restrict__ total)
{
    __shared__ uint32_t part[kColWarps][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int k = blockIdx.x * 32 + lane;
    const int per = (ctas + kColWarps - 1) / kColWarps;
    const int c0 = min(w * per, ctas), c1 = min(c0 + per, ctas);
    // rows are held in registers between the two passes (<= 32 per warp: ctas <= 256;
    // larger row counts take the slow path below)
    constexpr int kMaxRows = 32;
    uint32_t v[kMaxRows];
    uint32_t sum = 0;
    const bool fast = (c1 - c0) <= kMaxRows;
    if (k < K) {
        if (fast) {
#pragma unroll
            for (int u = 0; u < kMaxRows; u++)
                v[u] = (c0 + u < c1) ? hist[(int64_t)(c0 + u) * K + k] : 0u;
#pragma unroll
            for (int u = 0; u < kMaxRows; u++)
                sum += v[u];
        } else {
            for (int c = c0; c < c1; c++)
                sum += hist[(int64_t)c * K + k];
        }
    }
    part[w][lane] = sum;
    __syncthreads();
    uint32_t off = 0;
    for (int v = 0; v < w; v++)
        off += part[v][lane];
    if (w == kColWarps - 1 && k < K)
        total[k] = off + sum;
    if (k < K) {
        if (fast) {
#pragma unroll
            for (int u = 0; u < kMaxRows; u++)
                if (c0 + u < c1) {
                    hist[(int64_t)(c0 + u) * K + k] = off;
                    off += v[u];
                }
        } else {
            for (int c = c0; c < c1; c++) {
                const uint32_t x = hist[(int64_t)c * K + k];
                hist[(int64_t)c * K + k] = off;
                off += x;
            }
        }
    }
}

// one CTA: exclusive scan of base[0..K) in place.  Warp w owns a contiguous segment and
// walks it 32 coalesced elements at a time (warp scan + carry) -- no bank conflicts;
// a block scan of the warp totals gives each warp its offset for the second pass.  Then
// base[K + m] = first slot of material m, base[K + 12] = count.
__global__ void __launch_bounds__(1024) k_bucket_base(BucketPlan bp, uint32_t *__restrict__ base)
{
    __shared__ uint32_t wsum[32];
    const int K = bp.K;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int seg = ((K + 31) / 32 + 31) / 32 * 32; // elements per warp, multiple of 32
    const int b0 = min(wid * seg, K), b1 = min(b0 + seg, K);
    uint32_t tot = 0;
    for (int k = b0 + lane; k < b1; k += 32)
        tot += base[k];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
        tot += __shfl_xor_sync(0xffffffffu, tot, o);
    if (lane == 0)
        wsum[wid] = tot;
    __syncthreads();
    if (wid == 0) {
        uint32_t v = wsum[lane];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o)
                v += t;
        }
        wsum[lane] = v; // inclusive
    }
    __syncthreads();
    uint32_t carry = wid ? wsum[wid - 1] : 0u;
    for (int r = b0; r < b1; r += 32) {
        const int k = r + lane;
        const uint32_t v = k < b1 ? base[k] : 0u;
        uint32_t incl = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o)
                incl += t;
        }
        if (k < b1)
            base[k] = carry + incl - v;
        carry += __shfl_sync(0xffffffffu, incl, 31);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
#pragma unroll
        for (int m = 0; m < kMaterials; m++)
            base[K + m] = base[bp.kbase[m]];
        base[K + kMaterials] = wsum[31];
    }
}

__global__ void __launch_bounds__(kSortTpb) k_bucket_scatter(int K, int per_cta, int count,
                                                              const uint32_t *__restrict__ hist,
                                                              const uint32_t *__restrict__ base,
                                                              const uint16_t *__restrict__ key_of,
                                                              uint32_t *__restrict__ slot_of)
{
    extern __shared__ uint32_t sh[];
    const uint32_t *h = hist + (int64_t)blockIdx.x * K;
    for (int k = threadIdx.x; k < K; k += kSortTpb)
        sh[k] = base[k] + h[k];
    __syncthreads();
    const int beg = blockIdx.x * per_cta;
    const int end = min(beg + per_cta, count);
    // 4 keys in flight per thread, then their shared-memory atomics and 4 B stores
    // (recording each lookup's rank in the count pass to drop the atomics was measured
    // slower)
    int j = beg + threadIdx.x;
    for (; j + 3 * kSortTpb < end; j += 4 * kSortTpb) {
        uint32_t kk[4];
#pragma unroll
        for (int u = 0; u < 4; u++)
            kk[u] = key_of[j + u * kSortTpb];
#pragma unroll
        for (int u = 0; u < 4; u++)
            slot_of[atomicAdd(&sh[kk[u]], 1u)] = (uint32_t)(j + u * kSortTpb);
    }
    for (; j < end; j += kSortTpb)
        slot_of[atomicAdd(&sh[key_of[j]], 1u)] = (uint32_t)j;
}

__global__ void k_bucket_gather(int count, const uint32_t *__restrict__ slot_of, const double *__restrict__ q_of,
                                double *__restrict__ q_sorted)
{
    for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < count; j += gridDim.x * blockDim.x)
        q_sorted[j] = __ldg(q_of + __ldg(slot_of + j));
}

static int sm_count_dev()
{
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return sms > 0 ? sms : 148;
}

static void ensure_sort_space(Grid &g, int64_t chunk, int ctas, int K)
{
    if (g.cap < chunk) {
        cudaFree(g.sq);
        cudaFree(g.si);
        cudaFree(g.skey);
        cudaFree(g.qs);
        g.sq = g.qs = nullptr;
        g.si = nullptr;
        g.skey = nullptr;
        g.cap = 0;
        XS_CUDA_TRY(cudaMalloc(&g.sq, (size_t)chunk * sizeof(double)));
        XS_CUDA_TRY(cudaMalloc(&g.qs, (size_t)chunk * sizeof(double)));
        XS_CUDA_TRY(cudaMalloc(&g.si, (size_t)chunk * sizeof(uint32_t)));
        XS_CUDA_TRY(cudaMalloc(&g.skey, (size_t)chunk * sizeof(uint16_t)));
        g.cap = chunk;
    }
    const int64_t need = (int64_t)ctas * K;
    if (g.hist_cap < need) {
        cudaFree(g.hist);
        cudaFree(g.base);
        g.hist = nullptr;
        g.base = nullptr;
        g.hist_cap = 0;
        XS_CUDA_TRY(cudaMalloc(&g.hist, (size_t)need * sizeof(uint32_t)));
        XS_CUDA_TRY(cudaMalloc(&g.base, (size_t)(kMaterials * kMaxEnergyBins + 32) * sizeof(uint32_t)));
        g.hist_cap = need;
    }
}

static BucketPlan make_plan(const Grid &g, int nb_avg)
{
    BucketPlan bp{};
    double w[kMaterials], W = 0;
    for (int m = 0; m < kMaterials; m++) {
        const double p = (m == 0) ? 1.0 - g.thresholds[11] : g.thresholds[m] - g.thresholds[m - 1];
        w[m] = p * g.num_nucs[m];
        W += w[m];
    }
    // floor(total * share) + at most one bump to 1 per material stays <= 12 * nb_avg
    const int total = nb_avg > 1 ? kMaterials * (nb_avg - 1) : 0;
    int k = 0;
    for (int m = 0; m < kMaterials; m++) {
        bp.kbase[m] = k;
        bp.nb[m] = std::max(1, (int)(total * w[m] / W));
        k += bp.nb[m];
    }
    bp.kbase[kMaterials] = k;
    bp.K = k;
    return bp;
}

int launch_bucket_sort(Grid &g, const SampleView &sv, int nb_avg, bool with_gather, cudaStream_t stream, int *K_out)
{
    static bool smem_set[64] = {};
    if (!smem_set[g.device & 63]) {
        const int bytes = kMaterials * kMaxEnergyBins * 4;
        XS_CUDA_TRY(cudaFuncSetAttribute(k_bucket_count, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
        XS_CUDA_TRY(cudaFuncSetAttribute(k_bucket_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
        smem_set[g.device & 63] = true;
    }
    const int64_t cn = sv.count;
    const BucketPlan bp = make_plan(g, nb_avg);
    const int K = bp.K;
    *K_out = K;
    const int sms = sm_count_dev();
    const int ctas = (int)std::max<int64_t>(1, std::min<int64_t>(sms, (cn + kSortTpb - 1) / kSortTpb));
    const int per_cta = (int)((cn + ctas - 1) / ctas);
    ensure_sort_space(g, cn, ctas, K);
    const Affine J = lcg_jump(2 * (uint64_t)kSortTpb);
    const size_t smem = (size_t)K * 4;
    k_bucket_count<<<ctas, kSortTpb, smem, stream>>>(sv, bp, per_cta, J, g.hist, g.sq, g.skey);
    k_bucket_colscan<<<(K + 31) / 32, 32 * kColWarps, 0, stream>>>(K, ctas, g.hist, g.base);
    k_bucket_base<<<1, 1024, 0, stream>>>(bp, g.base);
    k_bucket_scatter<<<ctas, kSortTpb, smem, stream>>>(K, per_cta, (int)cn, g.hist, g.base, g.skey, g.si);
    XS_CUDA_TRY(cudaGetLastError());
    if (!with_gather)
        return 4;
    const int gblocks = (int)std::min<int64_t>((cn + 255) / 256, (int64_t)sms * 8);
    k_bucket_gather<<<gblocks, 256, 0, stream>>>((int)cn, g.si, g.sq, g.qs);
    XS_CUDA_TRY(cudaGetLastError());
    return 5;
}

} // namespace xs
