// lookup.cu -- the timed hot path (SURVEY.md §8a-2 .. a-7).
//
//   k_bucket_count   sample (q, mat) for a contiguous chunk of lookups per CTA and
//                    histogram the (material, energy-bucket) keys in shared memory
//   k_bucket_colscan per-bucket exclusive scan across CTAs
//   k_bucket_base    exclusive scan of the bucket totals (one CTA) + material bases
//   k_bucket_scatter re-sample (cheaper than storing) and scatter (q, i) to its slot
//   k_lookup         per lookup: per nuclide, search -> interpolate -> accumulate;
//                    argmax; fused CTA reduction of (hash, pairs) + one atomic per CTA
//
// With XS_SORT_NONE the sampling is fused into k_lookup (XSBench's baseline order).
// Every kernel here is templated on nothing but what changes its inner loop: the grid
// type, the search variant and whether lookups arrive sorted.
#include <algorithm>

#include "search.cuh"
#include "xs_internal.cuh"

namespace xs {

// ---- sampling -------------------------------------------------
// `s` is skip(seed, 2i); draws q at stream position 2i and the pick_mat roll at 2i+1.
__device__ __forceinline__ void sample_lookup(uint64_t s, const SampleView &sv, double &q, int &mat)
{
    uint64_t t = lcg_step(s);
    q = u63_to_double(t);
    t = lcg_step(t);
    const double roll = u63_to_double(t);
    // pick_mat (R9): the first m in 1..11 with roll < T[m], else 0 (T is increasing)
    int m = 0;
#pragma unroll
    for (int k = 11; k >= 1; k--)
        m = (roll < sv.T[k]) ? k : m;
    mat = m;
}

__device__ __forceinline__ uint64_t lookup_state(const SampleView &sv, int64_t j)
{
    return lcg_apply(lcg_jump(2 * (uint64_t)(sv.first + j)), sv.seed);
}

__device__ __forceinline__ int energy_bucket(double q, int nb_log2)
{
    const int nb = 1 << nb_log2;
    int b = (int)__dmul_rn(q, (double)nb); // exact: nb is a power of two
    return b < nb - 1 ? b : nb - 1;        // q may be exactly 1.0 (R7)
}

// ---- bucket sort ---------------------------------------------------------------------------
constexpr int kSortTpb = 1024;

__global__ void __launch_bounds__(kSortTpb) k_bucket_count(SampleView sv, int nb_log2, int64_t per_cta,
                                                            Affine J_tpb, uint32_t *__restrict__ hist)
{
    extern __shared__ uint32_t sh[];
    const int K = kMaterials << nb_log2;
    for (int k = threadIdx.x; k < K; k += kSortTpb)
        sh[k] = 0;
    __syncthreads();
    const int64_t beg = blockIdx.x * per_cta;
    const int64_t end = min(beg + per_cta, sv.count);
    int64_t j = beg + threadIdx.x;
    if (j < end) {
        uint64_t s = lookup_state(sv, j);
        for (; j < end; j += kSortTpb) {
            double q;
            int mat;
            sample_lookup(s, sv, q, mat);
            atomicAdd(&sh[(mat << nb_log2) + energy_bucket(q, nb_log2)], 1u);
            s = lcg_apply(J_tpb, s);
        }
    }
    __syncthreads();
    uint32_t *h = hist + (int64_t)blockIdx.x * K;
    for (int k = threadIdx.x; k < K; k += kSortTpb)
        h[k] = sh[k];
}

__global__ void k_bucket_colscan(int K, int ctas, uint32_t *__restrict__ hist, uint32_t *__restrict__ total)
{
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= K)
        return;
    uint32_t run = 0;
    for (int c = 0; c < ctas; c++) {
        const uint32_t v = hist[(int64_t)c * K + k];
        hist[(int64_t)c * K + k] = run;
        run += v;
    }
    total[k] = run;
}

// one CTA of 1024 threads: exclusive scan of total[0..K) in place; base[K + m] = start
// of material m (m = 0..12, base[K+12] = count)
__global__ void __launch_bounds__(1024) k_bucket_base(int K, int nb_log2, uint32_t *__restrict__ base)
{
    __shared__ uint32_t warp_sums[32];
    const int per = (K + 1023) / 1024;
    const int beg = threadIdx.x * per;
    const int end = min(beg + per, K);
    uint32_t local = 0;
    for (int k = beg; k < end; k++)
        local += base[k];
    // block exclusive scan of `local`
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t incl = local;
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o)
            incl += v;
    }
    if (lane == 31)
        warp_sums[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        uint32_t w = warp_sums[lane];
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t v = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o)
                w += v;
        }
        warp_sums[lane] = w; // inclusive
    }
    __syncthreads();
    uint32_t run = incl - local + (wid > 0 ? warp_sums[wid - 1] : 0);
    for (int k = beg; k < end; k++) {
        const uint32_t v = base[k];
        base[k] = run;
        run += v;
    }
    __syncthreads();
    if (threadIdx.x < kMaterials)
        base[K + threadIdx.x] = base[threadIdx.x << nb_log2];
    if (threadIdx.x == 0)
        base[K + kMaterials] = warp_sums[31];
}

__global__ void __launch_bounds__(kSortTpb) k_bucket_scatter(SampleView sv, int nb_log2, int64_t per_cta,
                                                              Affine J_tpb, const uint32_t *__restrict__ hist,
                                                              const uint32_t *__restrict__ base,
                                                              double *__restrict__ sq, uint32_t *__restrict__ si)
{
    extern __shared__ uint32_t sh[];
    const int K = kMaterials << nb_log2;
    const uint32_t *h = hist + (int64_t)blockIdx.x * K;
    for (int k = threadIdx.x; k < K; k += kSortTpb)
        sh[k] = base[k] + h[k];
    __syncthreads();
    const int64_t beg = blockIdx.x * per_cta;
    const int64_t end = min(beg + per_cta, sv.count);
    int64_t j = beg + threadIdx.x;
    if (j < end) {
        uint64_t s = lookup_state(sv, j);
        for (; j < end; j += kSortTpb) {
            double q;
            int mat;
            sample_lookup(s, sv, q, mat);
            const uint32_t pos = atomicAdd(&sh[(mat << nb_log2) + energy_bucket(q, nb_log2)], 1u);
            sq[pos] = q;
            si[pos] = (uint32_t)j;
            s = lcg_apply(J_tpb, s);
        }
    }
}

// ---- the lower index of one (lookup, nuclide) pair ----------------------
template <int GRID, int SEARCH>
__device__ __forceinline__ int lower_index(const GridView &gv, const double *__restrict__ Ei, int nuc, double q,
                                           int e_union)
{
    if constexpr (GRID == XS_NUCLIDE) {
        return search<SEARCH>(Ei, 0, gv.n - 1, q);
    } else if constexpr (GRID == XS_UNIONIZED) {
        return __ldg(gv.IDX + (int64_t)e_union * gv.n_nuc + nuc);
    } else { // hash window with guards (R7)
        int64_t b = (int64_t)__ddiv_rn(q, gv.du);
        b = b < 0 ? 0 : (b > gv.bins - 1 ? gv.bins - 1 : b);
        const int lo = __ldg(gv.H + b * gv.n_nuc + nuc);
        const int hi = (b == gv.bins - 1) ? gv.n - 1 : __ldg(gv.H + (b + 1) * gv.n_nuc + nuc) + 1;
        if (q < __ldg(Ei + lo) || (hi < gv.n - 1 && q >= __ldg(Ei + hi)))
            return search<SEARCH>(Ei, 0, gv.n - 1, q);
        return search<SEARCH>(Ei, lo, hi, q);
    }
}

template <int GRID, int SEARCH>
__device__ __forceinline__ int union_index(const GridView &gv, double q)
{
    if constexpr (GRID == XS_UNIONIZED)
        return search<SEARCH>(gv.U, 0, gv.N - 1, q);
    else
        return 0;
}

// ---- the lookup kernel ------------------------------------------------------------------------
constexpr int kLookupMaxTpb = 256;

template <int GRID, int SEARCH, bool SORTED>
__global__ void __launch_bounds__(kLookupMaxTpb)
    k_lookup(GridView gv, SampleView sv, Affine J_grid, const double *__restrict__ sq, const uint32_t *__restrict__ si,
             const uint32_t *__restrict__ matbase, double *__restrict__ out, int32_t *__restrict__ out_idx,
             unsigned long long *__restrict__ stats)
{
    __shared__ uint32_t s_matbase[kMaterials];
    __shared__ unsigned long long s_red[2][kLookupMaxTpb / 32];
    if constexpr (SORTED) {
        if (threadIdx.x < kMaterials)
            s_matbase[threadIdx.x] = matbase[threadIdx.x];
        __syncthreads();
    }
    uint64_t my_hash = 0, my_pairs = 0;
    const int64_t G = (int64_t)gridDim.x * blockDim.x;
    int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    uint64_t s = 0;
    if constexpr (!SORTED) {
        if (j < sv.count)
            s = lookup_state(sv, j);
    }
    for (; j < sv.count; j += G) {
        double q;
        int mat;
        int64_t r;
        if constexpr (SORTED) {
            q = sq[j];
            r = si[j];
            mat = 0;
#pragma unroll
            for (int m = 1; m < kMaterials; m++)
                mat += (j >= (int64_t)s_matbase[m]) ? 1 : 0;
        } else {
            sample_lookup(s, sv, q, mat);
            r = j;
            s = lcg_apply(J_grid, s);
        }
        const int nn = __ldg(gv.num_nucs + mat);
        const int32_t *__restrict__ mrow = gv.mats + mat * gv.max_nucs;
        const double *__restrict__ crow = gv.concs + mat * gv.max_nucs;
        const int e_union = union_index<GRID, SEARCH>(gv, q);
        double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0, a4 = 0.0;
        for (int jn = 0; jn < nn; jn++) {
            const int nuc = __ldg(mrow + jn);
            const double conc = __ldg(crow + jn);
            const double *__restrict__ Ei = gv.E + (int64_t)nuc * gv.n;
            const int L = lower_index<GRID, SEARCH>(gv, Ei, nuc, q, e_union);
            if (out_idx)
                out_idx[r * gv.max_nucs + jn] = L;
            // 96 B gather: the records of points L and L+1 (R8 arithmetic below)
            const double2 *p = reinterpret_cast<const double2 *>(gv.pts + ((int64_t)nuc * gv.n + L) * 6);
            const double2 l0 = __ldg(p + 0), l1 = __ldg(p + 1), l2 = __ldg(p + 2);
            const double2 h0 = __ldg(p + 3), h1 = __ldg(p + 4), h2 = __ldg(p + 5);
            const double f = __ddiv_rn(__dsub_rn(h0.x, q), __dsub_rn(h0.x, l0.x));
            a0 = __fma_rn(__fma_rn(-f, __dsub_rn(h0.y, l0.y), h0.y), conc, a0);
            a1 = __fma_rn(__fma_rn(-f, __dsub_rn(h1.x, l1.x), h1.x), conc, a1);
            a2 = __fma_rn(__fma_rn(-f, __dsub_rn(h1.y, l1.y), h1.y), conc, a2);
            a3 = __fma_rn(__fma_rn(-f, __dsub_rn(h2.x, l2.x), h2.x), conc, a3);
            a4 = __fma_rn(__fma_rn(-f, __dsub_rn(h2.y, l2.y), h2.y), conc, a4);
        }
        // verification (R10): first maximum, strict '>' from -1.0
        double mx = -1.0;
        int v = 0;
        if (a0 > mx) { mx = a0; v = 0; }
        if (a1 > mx) { mx = a1; v = 1; }
        if (a2 > mx) { mx = a2; v = 2; }
        if (a3 > mx) { mx = a3; v = 3; }
        if (a4 > mx) { mx = a4; v = 4; }
        my_hash += (uint64_t)(v + 1);
        my_pairs += (uint64_t)nn;
        if (out) {
            double *o = out + r * 5;
            o[0] = a0;
            o[1] = a1;
            o[2] = a2;
            o[3] = a3;
            o[4] = a4;
        }
    }
    // fused epilogue: CTA reduction, one atomic per counter per CTA
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        my_hash += __shfl_down_sync(0xffffffffu, my_hash, o);
        my_pairs += __shfl_down_sync(0xffffffffu, my_pairs, o);
    }
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) {
        s_red[0][wid] = my_hash;
        s_red[1][wid] = my_pairs;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long h = 0, pr = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            h += s_red[0][w];
            pr += s_red[1][w];
        }
        atomicAdd(stats + 0, h);
        atomicAdd(stats + 1, pr);
    }
}

// ---- debug kernels -------------------------------------------------------------------------
__global__ void k_sample(SampleView sv, double *__restrict__ q_out, int32_t *__restrict__ mat_out)
{
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < sv.count;
         j += (int64_t)gridDim.x * blockDim.x) {
        double q;
        int mat;
        sample_lookup(lookup_state(sv, j), sv, q, mat);
        q_out[j] = q;
        mat_out[j] = mat;
    }
}

template <int GRID, int SEARCH>
__global__ void k_search_points(GridView gv, int64_t count, const double *__restrict__ q,
                                const int32_t *__restrict__ nuc, int32_t *__restrict__ out)
{
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < count; t += (int64_t)gridDim.x * blockDim.x) {
        const double qq = q[t];
        const int nu = nuc[t];
        out[t] = lower_index<GRID, SEARCH>(gv, gv.E + (int64_t)nu * gv.n, nu, qq, union_index<GRID, SEARCH>(gv, qq));
    }
}

// ---- host side -------------------------------------------------------------------------------
static int sm_count()
{
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0)
            sms = 148;
    }
    return sms;
}

using LookupFn = void (*)(GridView, SampleView, Affine, const double *, const uint32_t *, const uint32_t *, double *,
                          int32_t *, unsigned long long *);
using SearchFn = void (*)(GridView, int64_t, const double *, const int32_t *, int32_t *);

template <int GRID, int SEARCH> static LookupFn pick_lookup_s(bool sorted)
{
    return sorted ? k_lookup<GRID, SEARCH, true> : k_lookup<GRID, SEARCH, false>;
}

template <int GRID> static LookupFn pick_lookup_g(int search, bool sorted)
{
    switch (search) {
    case XS_SEARCH_M: return pick_lookup_s<GRID, XS_SEARCH_M>(sorted);
    case XS_SEARCH_U1: return pick_lookup_s<GRID, XS_SEARCH_U1>(sorted);
    case XS_SEARCH_U2: return pick_lookup_s<GRID, XS_SEARCH_U2>(sorted);
    case XS_SEARCH_U4: return pick_lookup_s<GRID, XS_SEARCH_U4>(sorted);
    case XS_SEARCH_U8: return pick_lookup_s<GRID, XS_SEARCH_U8>(sorted);
    case XS_SEARCH_B: return pick_lookup_s<GRID, XS_SEARCH_B>(sorted);
    case XS_SEARCH_M2: return pick_lookup_s<GRID, XS_SEARCH_M2>(sorted);
    case XS_SEARCH_M4: return pick_lookup_s<GRID, XS_SEARCH_M4>(sorted);
    default: return pick_lookup_s<GRID, XS_SEARCH_M8>(sorted);
    }
}

static LookupFn pick_lookup(int grid_type, int search, bool sorted)
{
    if (grid_type == XS_NUCLIDE)
        return pick_lookup_g<XS_NUCLIDE>(search, sorted);
    if (grid_type == XS_UNIONIZED)
        return pick_lookup_g<XS_UNIONIZED>(search, sorted);
    return pick_lookup_g<XS_HASH>(search, sorted);
}

template <int GRID> static SearchFn pick_search_g(int search)
{
    switch (search) {
    case XS_SEARCH_M: return k_search_points<GRID, XS_SEARCH_M>;
    case XS_SEARCH_U1: return k_search_points<GRID, XS_SEARCH_U1>;
    case XS_SEARCH_U2: return k_search_points<GRID, XS_SEARCH_U2>;
    case XS_SEARCH_U4: return k_search_points<GRID, XS_SEARCH_U4>;
    case XS_SEARCH_U8: return k_search_points<GRID, XS_SEARCH_U8>;
    case XS_SEARCH_B: return k_search_points<GRID, XS_SEARCH_B>;
    case XS_SEARCH_M2: return k_search_points<GRID, XS_SEARCH_M2>;
    case XS_SEARCH_M4: return k_search_points<GRID, XS_SEARCH_M4>;
    default: return k_search_points<GRID, XS_SEARCH_M8>;
    }
}

static SearchFn pick_search(int grid_type, int search)
{
    if (grid_type == XS_NUCLIDE)
        return pick_search_g<XS_NUCLIDE>(search);
    if (grid_type == XS_UNIONIZED)
        return pick_search_g<XS_UNIONIZED>(search);
    return pick_search_g<XS_HASH>(search);
}

static void ensure_sort_space(Grid &g, int64_t chunk, int ctas, int K)
{
    if (g.cap < chunk) {
        cudaFree(g.sq);
        cudaFree(g.si);
        g.sq = nullptr;
        g.si = nullptr;
        g.cap = 0;
        XS_CUDA_TRY(cudaMalloc(&g.sq, (size_t)chunk * sizeof(double)));
        XS_CUDA_TRY(cudaMalloc(&g.si, (size_t)chunk * sizeof(uint32_t)));
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

static bool is_device_accessible(const void *p)
{
    cudaPointerAttributes a{};
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

static int log2_exact(int v)
{
    int l = 0;
    while ((1 << l) < v)
        l++;
    return ((1 << l) == v) ? l : -1;
}

// Largest lookups per internal pass: positions are uint32 and scratch stays bounded.
constexpr int64_t kChunkDevice = int64_t(1) << 28;
constexpr int64_t kChunkHost = int64_t(1) << 23;

void run_lookups(Grid &g, int64_t first, int64_t count, uint64_t seed, const xs_opts &o, double *out_macro,
                 int32_t *out_idx, xs_stats *st)
{
    XS_CHECK_ARG(o.search >= 0 && o.search < XS_SEARCH_COUNT, "opts.search out of range");
    XS_CHECK_ARG(o.sort >= XS_SORT_NONE && o.sort <= XS_SORT_MATERIAL_ENERGY, "opts.sort out of range");
    const int tpb = o.block ? o.block : 256;
    XS_CHECK_ARG(tpb == 64 || tpb == 128 || tpb == 256, "opts.block must be 64, 128 or 256");
    int nb = (o.sort == XS_SORT_MATERIAL_ENERGY) ? (o.energy_bins ? o.energy_bins : kMaxEnergyBins) : 1;
    const int nb_log2 = log2_exact(nb);
    XS_CHECK_ARG(nb_log2 >= 0 && nb <= kMaxEnergyBins, "opts.energy_bins must be a power of two <= 4096");
    cudaStream_t stream = (cudaStream_t)o.stream;
    const bool timing = (o.flags & XS_FLAG_TIMING) != 0;

    const bool host_out = out_macro && !is_device_accessible(out_macro);
    const int64_t chunk_max = host_out ? kChunkHost : kChunkDevice;
    const bool sorted = o.sort != XS_SORT_NONE;
    const int K = kMaterials << nb_log2;
    const int sms = sm_count();
    const GridView gv = make_view(g);
    const LookupFn kfn = pick_lookup(g.grid_type, o.search, sorted);
    int launches = 0;
    double sample_ms = 0, lookup_ms = 0, copy_ms = 0;

    if (host_out && g.stage_cap < std::min(count, chunk_max)) {
        cudaFree(g.stage);
        g.stage = nullptr;
        g.stage_cap = 0;
        const int64_t c = std::min(count, chunk_max);
        XS_CUDA_TRY(cudaMalloc(&g.stage, (size_t)c * 5 * sizeof(double)));
        g.stage_cap = c;
    }
    static bool smem_set[64] = {};
    if (!smem_set[g.device & 63]) {
        const int bytes = kMaterials * kMaxEnergyBins * 4;
        XS_CUDA_TRY(cudaFuncSetAttribute(k_bucket_count, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
        XS_CUDA_TRY(cudaFuncSetAttribute(k_bucket_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
        smem_set[g.device & 63] = true;
    }

    XS_CUDA_TRY(cudaEventRecord(g.ev[0], stream));
    XS_CUDA_TRY(cudaMemsetAsync(g.stats_d, 0, 2 * sizeof(uint64_t), stream));
    if (out_idx && count > 0)
        XS_CUDA_TRY(cudaMemsetAsync(out_idx, 0xFF, (size_t)count * g.max_nucs * sizeof(int32_t), stream));

    for (int64_t c0 = 0; c0 < count; c0 += chunk_max) {
        const int64_t cn = std::min(chunk_max, count - c0);
        SampleView sv = make_sample_view(g, seed, first + c0, cn);
        const uint32_t *matbase = nullptr;
        if (timing)
            XS_CUDA_TRY(cudaEventRecord(g.ev[1], stream));
        if (sorted) {
            const int ctas = (int)std::max<int64_t>(1, std::min<int64_t>(sms, (cn + kSortTpb - 1) / kSortTpb));
            const int64_t per_cta = (cn + ctas - 1) / ctas;
            ensure_sort_space(g, std::min(count, chunk_max), ctas, K);
            const Affine J = lcg_jump(2 * (uint64_t)kSortTpb);
            const size_t smem = (size_t)K * 4;
            k_bucket_count<<<ctas, kSortTpb, smem, stream>>>(sv, nb_log2, per_cta, J, g.hist);
            k_bucket_colscan<<<(K + 255) / 256, 256, 0, stream>>>(K, ctas, g.hist, g.base);
            k_bucket_base<<<1, 1024, 0, stream>>>(K, nb_log2, g.base);
            k_bucket_scatter<<<ctas, kSortTpb, smem, stream>>>(sv, nb_log2, per_cta, J, g.hist, g.base, g.sq, g.si);
            XS_CUDA_TRY(cudaGetLastError());
            matbase = g.base + K;
            launches += 4;
        }
        if (timing)
            XS_CUDA_TRY(cudaEventRecord(g.ev[2], stream));
        const int resident = 2048 / tpb;
        const int64_t want = (cn + tpb - 1) / tpb;
        const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)sms * resident * 4));
        const Affine Jg = lcg_jump(2 * (uint64_t)blocks * tpb);
        double *outp = out_macro ? (host_out ? g.stage : out_macro + c0 * 5) : nullptr;
        int32_t *idxp = out_idx ? out_idx + c0 * g.max_nucs : nullptr;
        kfn<<<blocks, tpb, 0, stream>>>(gv, sv, Jg, g.sq, g.si, matbase, outp, idxp,
                                        (unsigned long long *)g.stats_d);
        XS_CUDA_TRY(cudaGetLastError());
        launches += 1;
        if (timing)
            XS_CUDA_TRY(cudaEventRecord(g.ev[3], stream));
        if (host_out) {
            XS_CUDA_TRY(cudaMemcpyAsync(out_macro + c0 * 5, g.stage, (size_t)cn * 5 * sizeof(double),
                                        cudaMemcpyDeviceToHost, stream));
            if (timing)
                XS_CUDA_TRY(cudaEventRecord(g.ev[4], stream));
        }
        if (timing) {
            XS_CUDA_TRY(cudaStreamSynchronize(stream));
            float a = 0, b = 0, c = 0;
            cudaEventElapsedTime(&a, g.ev[1], g.ev[2]);
            cudaEventElapsedTime(&b, g.ev[2], g.ev[3]);
            if (host_out)
                cudaEventElapsedTime(&c, g.ev[3], g.ev[4]);
            sample_ms += a;
            lookup_ms += b;
            copy_ms += c;
        }
    }
    XS_CUDA_TRY(cudaMemcpyAsync(g.stats_h, g.stats_d, 2 * sizeof(uint64_t), cudaMemcpyDeviceToHost, stream));
    XS_CUDA_TRY(cudaEventRecord(g.ev[5], stream));
    XS_CUDA_TRY(cudaStreamSynchronize(stream));
    float total = 0;
    XS_CUDA_TRY(cudaEventElapsedTime(&total, g.ev[0], g.ev[5]));
    if (st) {
        st->hash = g.stats_h[0];
        st->pairs = g.stats_h[1];
        st->lookups = (uint64_t)count;
        st->device_ms = total;
        st->sample_ms = sample_ms;
        st->lookup_ms = lookup_ms;
        st->copy_ms = copy_ms;
        st->lookup_launches = launches;
    }
}

void run_sample(Grid &g, int64_t first, int64_t count, uint64_t seed, double *q, int32_t *mat, cudaStream_t s)
{
    if (count == 0)
        return;
    SampleView sv = make_sample_view(g, seed, first, count);
    const int blocks = (int)std::min<int64_t>((count + 255) / 256, 148 * 32);
    k_sample<<<blocks, 256, 0, s>>>(sv, q, mat);
    XS_CUDA_TRY(cudaGetLastError());
    XS_CUDA_TRY(cudaStreamSynchronize(s));
}

void run_search_points(Grid &g, int64_t count, const double *q, const int32_t *nuc, int search, int32_t *out,
                       cudaStream_t s)
{
    XS_CHECK_ARG(search >= 0 && search < XS_SEARCH_COUNT, "search out of range");
    if (count == 0)
        return;
    const int blocks = (int)std::min<int64_t>((count + 255) / 256, 148 * 32);
    pick_search(g.grid_type, search)<<<blocks, 256, 0, s>>>(make_view(g), count, q, nuc, out);
    XS_CUDA_TRY(cudaGetLastError());
    XS_CUDA_TRY(cudaStreamSynchronize(s));
}

} // namespace xs
