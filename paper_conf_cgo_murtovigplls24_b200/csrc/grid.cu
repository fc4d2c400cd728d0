// grid.cu -- grid generation and layout on the device.
//
// Setup, not timed (XSBench's grid_init_do_not_profile [XSB]; PAPER.md:244 excludes
// memcpy).  Steps:
//   k_fill_points   point p draws the stream positions 6p..6p+5 (energy + 5 channels);
//                   one Listing-7 jump per thread (rng.cuh)
//   segmented sort  per nuclide, ascending energy (CUB radix sort: a library sort, as
//                   the oracle uses qsort)
//   k_layout        E (SoA keys) + pts (48 B records); duplicate-energy check (R5)
//   unionized       U = radix sort of all energies; IDX[e][i] = Listing-1 search (R4)
//   hash            H[b][i] = Listing-1 search at b*du (R7)
#include <cub/cub.cuh>

#include <vector>

#include "search.cuh"
#include "xs_internal.cuh"

namespace xs {

// ---- material tables [XSB] (reading R9) ------------------------------
static const int32_t kFuelSmall[34] = {58, 59, 60, 61, 40, 42, 43, 44, 45, 46, 1,  2,  3,  7,  8,  9,  10,
                                       29, 57, 47, 48, 0,  62, 15, 33, 34, 52, 53, 54, 55, 56, 18, 23, 41};
static const int32_t kMat1[5] = {63, 64, 65, 66, 67};
static const int32_t kMat23[4] = {24, 41, 4, 5};
static const int32_t kMat4[27] = {19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 27, 28, 29, 30,
                                  31, 32, 26, 49, 50, 51, 11, 12, 13, 14, 6,  16, 17};
static const int32_t kMat59[21] = {24, 41, 4, 5, 19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 49, 50, 51, 11, 12, 13, 14};
static const int32_t kMat1011[9] = {24, 41, 4, 5, 63, 64, 65, 66, 67};
static const double kDist[12] = {0.140, 0.052, 0.275, 0.134, 0.154, 0.064,
                                 0.066, 0.055, 0.008, 0.015, 0.025, 0.013};

static void material_tables(Grid &g, std::vector<int32_t> &mats)
{
    const int32_t fuel = (g.n_nuc == 68) ? 34 : 321;
    const int32_t nn[12] = {fuel, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9};
    g.max_nucs = fuel;
    for (int m = 0; m < 12; m++)
        g.num_nucs[m] = nn[m];
    mats.assign((size_t)12 * fuel, -1);
    auto row = [&](int m) { return mats.data() + (size_t)m * fuel; };
    for (int j = 0; j < 34; j++)
        row(0)[j] = kFuelSmall[j];
    for (int j = 34; j < fuel; j++)
        row(0)[j] = 68 + (j - 34);
    for (int j = 0; j < 5; j++)
        row(1)[j] = kMat1[j];
    for (int m = 2; m <= 3; m++)
        for (int j = 0; j < 4; j++)
            row(m)[j] = kMat23[j];
    for (int j = 0; j < 27; j++)
        row(4)[j] = kMat4[j];
    for (int m = 5; m <= 9; m++)
        for (int j = 0; j < 21; j++)
            row(m)[j] = kMat59[j];
    for (int m = 10; m <= 11; m++)
        for (int j = 0; j < 9; j++)
            row(m)[j] = kMat1011[j];
    // pick_mat running sums: T[i] = dist[i] + dist[i-1] + ... + dist[1], in that order
    for (int i = 0; i < 12; i++) {
        double running = 0;
        for (int j = i; j > 0; j--)
            running += kDist[j];
        g.thresholds[i] = running;
    }
}

// ---- kernels -------------------------------------------------------------------------
__global__ void k_fill_points(uint64_t seed, int64_t N, int32_t n, double *__restrict__ keys,
                              uint32_t *__restrict__ vals, double *__restrict__ raw)
{
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < N; p += (int64_t)gridDim.x * blockDim.x) {
        uint64_t s = lcg_apply(lcg_jump(6 * (uint64_t)p), seed);
        s = lcg_step(s);
        keys[p] = u63_to_double(s);
        vals[p] = (uint32_t)(p % n);
#pragma unroll
        for (int c = 0; c < 5; c++) {
            s = lcg_step(s);
            raw[p * 5 + c] = u63_to_double(s);
        }
    }
}

// the staged kernel's interval records (XS_S_TMA): ivs[i] for interval L = i mod (n-1) of
// nuclide i / (n-1), 14 doubles, rounded exactly as lookup_staged.cu's stage_interval rounds
// them (so results stay bit-identical); slot 1 (the concentration there) is 0 here
__global__ void k_ivs_build(int64_t NI, int32_t n, const double *__restrict__ pts, double *__restrict__ ivs)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NI; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t nuc = i / (n - 1), L = i - nuc * (n - 1);
        const double *lo = pts + (nuc * n + L) * 6, *hi = lo + 6;
        double *o = ivs + i * 14;
        const double d = __dsub_rn(hi[0], lo[0]);
        o[0] = hi[0];
        o[1] = 0.0;
        o[2] = d;
        o[3] = __drcp_rn(d);
#pragma unroll
        for (int c = 0; c < 5; c++) {
            o[4 + 2 * c] = hi[1 + c];
            o[5 + 2 * c] = __dsub_rn(hi[1 + c], lo[1 + c]);
        }
    }
}

// interval records (XS_IV): iv[i] for interval L = i mod (n-1) of nuclide i / (n-1)
__global__ void k_iv_build(int64_t NI, int32_t n, const double *__restrict__ pts, double *__restrict__ iv)
{
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < NI; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t nuc = i / (n - 1), L = i - nuc * (n - 1);
        const double *lo = pts + (nuc * n + L) * 6, *hi = lo + 6;
        double *o = iv + i * 12;
        o[0] = hi[0];
        o[1] = __dsub_rn(hi[0], lo[0]);
#pragma unroll
        for (int c = 0; c < 5; c++) {
            o[2 + 2 * c] = hi[1 + c];
            o[3 + 2 * c] = __dsub_rn(hi[1 + c], lo[1 + c]);
        }
    }
}

__global__ void k_layout(int64_t N, int32_t n, const double *__restrict__ keys, const uint32_t *__restrict__ vals,
                         const double *__restrict__ raw, double *__restrict__ E, double *__restrict__ pts,
                         int *__restrict__ dup)
{
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < N; p += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = p % n;
        const int64_t src = (p - r) + vals[p];
        const double e = keys[p];
        E[p] = e;
        double *o = pts + p * 6;
        o[0] = e;
#pragma unroll
        for (int c = 0; c < 5; c++)
            o[1 + c] = raw[src * 5 + c];
        if (r > 0 && !(e > keys[p - 1]))
            atomicOr(dup, 1);
    }
}

__global__ void k_segment_offsets(int64_t n_nuc, int32_t n, int *__restrict__ off)
{
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i <= n_nuc)
        off[i] = (int)(i * n);
}

__global__ void k_union_idx(int64_t total, int32_t n_nuc, int32_t n, const double *__restrict__ E,
                            const double *__restrict__ U, int32_t *__restrict__ IDX)
{
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t e = t / n_nuc;
        const int32_t i = (int32_t)(t - e * n_nuc);
        IDX[t] = search_M<1>(E + (int64_t)i * n, 0, n - 1, U[e]);
    }
}

__global__ void k_hash_table(int64_t bins, int32_t n_nuc, int32_t n, double du, const double *__restrict__ E,
                             int32_t *__restrict__ H)
{
    const int64_t total = bins * n_nuc;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = t / n_nuc;
        const int32_t i = (int32_t)(t - b * n_nuc);
        const double energy = __dmul_rn((double)b, du);
        H[t] = search_M<1>(E + (int64_t)i * n, 0, n - 1, energy);
    }
}

// separator tree: level d node `node` (path digits c_0..c_{d-1} in base 17) starts at
// base = sum c_k * stride[k]; its key t is E[base + (t+1)*stride[d]] or +inf past the row
__global__ void k_tree_build(int64_t n_nuc, int32_t n, int32_t levels, int4 stride_lo, int2 stride_hi,
                             int4 off_lo, int2 off_hi, int64_t per_nuc, const double *__restrict__ E,
                             double *__restrict__ keys)
{
    const int32_t stride[6] = {stride_lo.x, stride_lo.y, stride_lo.z, stride_lo.w, stride_hi.x, stride_hi.y};
    const int32_t off[6] = {off_lo.x, off_lo.y, off_lo.z, off_lo.w, off_hi.x, off_hi.y};
    const int64_t total = n_nuc * per_nuc;
    for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < total; g += (int64_t)gridDim.x * blockDim.x) {
        const int64_t nuc = g / per_nuc;
        const int32_t k = (int32_t)(g - nuc * per_nuc);
        int d = 0;
        while (d + 1 < levels && k >= off[d + 1])
            d++;
        const int32_t in_level = k - off[d];
        const int32_t node = in_level / kTreeFan, t = in_level % kTreeFan;
        int64_t base = 0;
        int32_t rest = node;
        for (int e = d - 1; e >= 0; e--) { // least significant digit = deepest level
            base += (int64_t)(rest % 17) * stride[e];
            rest /= 17;
        }
        const int64_t pos = base + (int64_t)(t + 1) * stride[d];
        keys[g] = pos < n ? E[nuc * n + pos] : __longlong_as_double(0x7FF0000000000000ll);
    }
}

// bin table: entry (nuc, b) = {L(b/2^k), L((b+1)/2^k) - L(b/2^k), E[L(b/2^k) + 1]} of the
// row (the energies b/2^k are exact in fp64)
__global__ void k_bins_build(int64_t n_nuc, int32_t n, int32_t b_log2, const double *__restrict__ E,
                             BinEntry *__restrict__ B)
{
    const int64_t per = (int64_t)1 << b_log2;
    const int64_t total = n_nuc * per;
    const double scale = 1.0 / (double)per;
    for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < total; g += (int64_t)gridDim.x * blockDim.x) {
        const int64_t nuc = g / per;
        const int64_t b = g - nuc * per;
        const double *row = E + nuc * n;
        const int lo = search_M<1>(row, 0, n - 1, __dmul_rn((double)b, scale));
        const int hi = search_M<1>(row, 0, n - 1, __dmul_rn((double)(b + 1), scale));
        BinEntry e;
        e.lo = lo;
        e.cnt = hi - lo;
        e.e_next = row[lo + 1 < n ? lo + 1 : n - 1];
        B[g] = e;
    }
}

// position-weighted checksum: h += word_k * (2*(offset+k)+1) over 32-bit words
__global__ void k_checksum(const uint32_t *__restrict__ w, int64_t nwords, uint64_t offset, unsigned long long *out)
{
    uint64_t h = 0;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nwords; k += (int64_t)gridDim.x * blockDim.x)
        h += (uint64_t)w[k] * (2 * (offset + (uint64_t)k) + 1);
    for (int o = 16; o > 0; o >>= 1)
        h += __shfl_down_sync(0xffffffffu, h, o);
    if ((threadIdx.x & 31) == 0)
        atomicAdd(out, (unsigned long long)h);
}

static int grid_blocks(int64_t work, int tpb)
{
    int64_t b = (work + tpb - 1) / tpb;
    if (b > 148 * 64)
        b = 148 * 64;
    return (int)(b < 1 ? 1 : b);
}

template <class T> static T *dalloc(Grid &g, int64_t count, bool owned = true)
{
    void *p = nullptr;
    XS_CUDA_TRY(cudaMalloc(&p, (size_t)count * sizeof(T)));
    if (owned)
        g.device_bytes += (uint64_t)count * sizeof(T);
    return (T *)p;
}

void build_grid(Grid &g)
{
    std::vector<int32_t> mats;
    material_tables(g, mats);
    const int64_t N = g.N;
    const int32_t n = (int32_t)g.n;
    const int tpb = 256;

    g.E = dalloc<double>(g, N);
    g.pts = dalloc<double>(g, N * 6);
    g.mats = dalloc<int32_t>(g, 12 * (int64_t)g.max_nucs);
    g.concs = dalloc<double>(g, 12 * (int64_t)g.max_nucs);
    g.num_nucs_d = dalloc<int32_t>(g, 12);

    // ---- nuclide grid: fill, per-nuclide sort, layout
    double *keys = nullptr, *keys_out = nullptr, *raw = nullptr;
    uint32_t *vals = nullptr, *vals_out = nullptr;
    int *offs = nullptr, *dup = nullptr;
    void *tmp = nullptr;
    auto cleanup = [&]() {
        cudaFree(keys);
        cudaFree(keys_out);
        cudaFree(raw);
        cudaFree(vals);
        cudaFree(vals_out);
        cudaFree(offs);
        cudaFree(dup);
        cudaFree(tmp);
        keys = keys_out = raw = nullptr;
        vals = vals_out = nullptr;
        offs = dup = nullptr;
        tmp = nullptr;
    };
    try {
        keys = dalloc<double>(g, N, false);
        keys_out = dalloc<double>(g, N, false);
        raw = dalloc<double>(g, N * 5, false);
        vals = dalloc<uint32_t>(g, N, false);
        vals_out = dalloc<uint32_t>(g, N, false);
        offs = dalloc<int>(g, g.n_nuc + 1, false);
        dup = dalloc<int>(g, 1, false);
        XS_CUDA_TRY(cudaMemset(dup, 0, sizeof(int)));

        k_fill_points<<<grid_blocks(N, tpb), tpb>>>(g.seed, N, n, keys, vals, raw);
        k_segment_offsets<<<(int)((g.n_nuc + 1 + 255) / 256), 256>>>(g.n_nuc, n, offs);
        XS_CUDA_TRY(cudaGetLastError());
        size_t tmp_bytes = 0;
        XS_CUDA_TRY(cub::DeviceSegmentedRadixSort::SortPairs(nullptr, tmp_bytes, keys, keys_out, vals, vals_out,
                                                             (int)N, (int)g.n_nuc, offs, offs + 1));
        XS_CUDA_TRY(cudaMalloc(&tmp, tmp_bytes));
        XS_CUDA_TRY(cub::DeviceSegmentedRadixSort::SortPairs(tmp, tmp_bytes, keys, keys_out, vals, vals_out,
                                                             (int)N, (int)g.n_nuc, offs, offs + 1));
        k_layout<<<grid_blocks(N, tpb), tpb>>>(N, n, keys_out, vals_out, raw, g.E, g.pts, dup);
        XS_CUDA_TRY(cudaGetLastError());
        if (kIv) {
            const int64_t NI = g.n_nuc * (n - 1);
            g.iv = dalloc<double>(g, NI * 12);
            k_iv_build<<<grid_blocks(NI, tpb), tpb>>>(NI, n, g.pts, g.iv);
            XS_CUDA_TRY(cudaGetLastError());
        }
        if (kTmaStage && g.grid_type == XS_HASH) { // the staged kernel's bulk-copied records (hash grid)
            const int64_t NI = g.n_nuc * (n - 1);
            g.ivs = dalloc<double>(g, NI * 14);
            k_ivs_build<<<grid_blocks(NI, tpb), tpb>>>(NI, n, g.pts, g.ivs);
            XS_CUDA_TRY(cudaGetLastError());
        }
        int dup_h = 0;
        XS_CUDA_TRY(cudaMemcpy(&dup_h, dup, sizeof(int), cudaMemcpyDeviceToHost));
        if (dup_h)
            throw Error{XS_EDUP, "duplicate energy within a nuclide (grid seed gives a tie)"};
        cudaFree(tmp);
        tmp = nullptr;

        // ---- separator tree over every nuclide row (XS_SEARCH_W; only the nuclide-grid
        // kernels read it: on XL's hash grid it would be ~0.24 GB never used)
        if (g.grid_type == XS_NUCLIDE) {
            int64_t R = n;
            g.t_levels = 0;
            int64_t nodes = 1, off = 0;
            while (R > kTreeFan) {
                const int64_t s = (R + 16) / 17; // ceil(R / 17)
                g.t_stride[g.t_levels] = (int32_t)s;
                g.t_off[g.t_levels] = (int32_t)off;
                off += nodes * kTreeFan;
                nodes *= 17;
                g.t_levels++;
                R = s;
            }
            g.t_leaf = (int32_t)R;
            g.t_per_nuc = off;
            if (off > 0) {
                g.tkeys = dalloc<double>(g, g.n_nuc * off);
                const int4 slo = make_int4(g.t_stride[0], g.t_stride[1], g.t_stride[2], g.t_stride[3]);
                const int2 shi = make_int2(g.t_stride[4], g.t_stride[5]);
                const int4 olo = make_int4(g.t_off[0], g.t_off[1], g.t_off[2], g.t_off[3]);
                const int2 ohi = make_int2(g.t_off[4], g.t_off[5]);
                k_tree_build<<<grid_blocks(g.n_nuc * off, tpb), tpb>>>(g.n_nuc, n, g.t_levels, slo, shi, olo, ohi,
                                                                      off, g.E, g.tkeys);
                XS_CUDA_TRY(cudaGetLastError());
            }
        }
        // ---- bin bounds over every nuclide row (XS_SEARCH_H / S on the nuclide grid only;
        // the unionized grid bounds its U search with ubnd, the hash grid uses H): 2^k >= n bins
        if (g.grid_type == XS_NUCLIDE) {
            int b_log2 = 1;
            while ((int64_t(1) << b_log2) < g.n && b_log2 < 20)
                b_log2++;
            // oversample (up to 4x) while the point records and the bin table still fit in
            // L2 together: fewer bins hold >= 2 points, so fewer pairs need a window probe
            // (small tables 1.045x; large tables, already past L2, keep 2^k >= n)
            int l2_bytes = 0;
            XS_CUDA_TRY(cudaDeviceGetAttribute(&l2_bytes, cudaDevAttrL2CacheSize, g.device));
            for (int extra = 0; extra < 2 && b_log2 < 22; extra++) {
                const int64_t bytes = g.N * 48 + g.n_nuc * (int64_t)sizeof(BinEntry) * (int64_t(1) << (b_log2 + 1));
                if (bytes > (int64_t)l2_bytes)
                    break;
                b_log2++;
            }
            const int64_t per = int64_t(1) << b_log2;
            if (g.n_nuc * per < (int64_t(1) << 31)) {
                g.b_log2 = b_log2;
                g.bnd = dalloc<BinEntry>(g, g.n_nuc * per);
                k_bins_build<<<grid_blocks(g.n_nuc * per, tpb), tpb>>>(g.n_nuc, n, b_log2, g.E, g.bnd);
                XS_CUDA_TRY(cudaGetLastError());
            }
        }
        // ---- unionized grid (R4)
        if (g.grid_type == XS_UNIONIZED) {
            g.U = dalloc<double>(g, N);
            tmp_bytes = 0;
            XS_CUDA_TRY(cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, g.E, g.U, (int)N));
            XS_CUDA_TRY(cudaMalloc(&tmp, tmp_bytes));
            XS_CUDA_TRY(cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, g.E, g.U, (int)N));
            // bin bounds of U (XS_SEARCH_H): UB[b] = Listing1(U, b / 2^k), 2^k >= N
            {
                int u_log2 = 1;
                while ((int64_t(1) << u_log2) < N && u_log2 < 26)
                    u_log2++;
                g.u_log2 = u_log2;
                g.ubnd = dalloc<BinEntry>(g, int64_t(1) << u_log2);
                k_bins_build<<<grid_blocks(int64_t(1) << u_log2, tpb), tpb>>>(1, (int32_t)N, u_log2, g.U, g.ubnd);
                XS_CUDA_TRY(cudaGetLastError());
            }
            g.IDX = dalloc<int32_t>(g, N * g.n_nuc);
            const int64_t total = N * g.n_nuc;
            k_union_idx<<<grid_blocks(total, tpb), tpb>>>(total, (int32_t)g.n_nuc, n, g.E, g.U, g.IDX);
            XS_CUDA_TRY(cudaGetLastError());
        }
        // ---- hash grid (R7)
        if (g.grid_type == XS_HASH) {
            g.H = dalloc<int32_t>(g, g.bins * g.n_nuc);
            const double du = 1.0 / (double)g.bins;
            k_hash_table<<<grid_blocks(g.bins * g.n_nuc, tpb), tpb>>>(g.bins, (int32_t)g.n_nuc, n, du, g.E, g.H);
            XS_CUDA_TRY(cudaGetLastError());
        }
        XS_CUDA_TRY(cudaDeviceSynchronize());
        cleanup();
    } catch (...) {
        cleanup();
        throw;
    }

    // ---- materials: concentrations continue the grid stream at 6N (R11)
    std::vector<double> concs((size_t)12 * g.max_nucs, 0.0);
    uint64_t t = 6 * (uint64_t)N;
    for (int m = 0; m < 12; m++)
        for (int j = 0; j < g.num_nucs[m]; j++) {
            uint64_t s = lcg_step(lcg_apply(lcg_jump(t++), g.seed));
            concs[(size_t)m * g.max_nucs + j] = u63_to_double_host(s);
        }
    XS_CUDA_TRY(cudaMemcpy(g.mats, mats.data(), mats.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
    XS_CUDA_TRY(cudaMemcpy(g.concs, concs.data(), concs.size() * sizeof(double), cudaMemcpyHostToDevice));
    XS_CUDA_TRY(cudaMemcpy(g.num_nucs_d, g.num_nucs, 12 * sizeof(int32_t), cudaMemcpyHostToDevice));
    {
        std::vector<NucRef> refs((size_t)12 * g.max_nucs, NucRef{nullptr, nullptr, nullptr, nullptr, 0.0, 0});
        static_assert(sizeof(NucRef) == 48, "NucRef is loaded as three 16 B vectors");
        for (int m = 0; m < 12; m++)
            for (int j = 0; j < g.num_nucs[m]; j++) {
                const int64_t nuc = mats[(size_t)m * g.max_nucs + j];
                NucRef &r = refs[(size_t)m * g.max_nucs + j];
                r.E = g.E + nuc * g.n;
                r.pts = kIv ? g.iv + nuc * (g.n - 1) * 12 : g.pts + nuc * g.n * 6;
                r.T = g.tkeys ? g.tkeys + nuc * g.t_per_nuc : nullptr;
                r.B = g.bnd ? g.bnd + nuc * (int64_t(1) << g.b_log2) : nullptr;
                r.conc = concs[(size_t)m * g.max_nucs + j];
                r.nuc = nuc;
            }
        g.refs = dalloc<NucRef>(g, (int64_t)refs.size());
        XS_CUDA_TRY(cudaMemcpy(g.refs, refs.data(), refs.size() * sizeof(NucRef), cudaMemcpyHostToDevice));
    }

    XS_CUDA_TRY(cudaMalloc(&g.stats_d, 8 * sizeof(uint64_t)));
    XS_CUDA_TRY(cudaMallocHost(&g.stats_h, 8 * sizeof(uint64_t)));
    for (auto &e : g.ev)
        XS_CUDA_TRY(cudaEventCreate(&e));
}

void free_grid(Grid &g)
{
    cudaFree(g.E);
    cudaFree(g.pts);
    cudaFree(g.iv);
    cudaFree(g.ivs);
    cudaFree(g.tkeys);
    cudaFree(g.bnd);
    cudaFree(g.ubnd);
    cudaFree(g.U);
    cudaFree(g.IDX);
    cudaFree(g.H);
    cudaFree(g.mats);
    cudaFree(g.concs);
    cudaFree(g.num_nucs_d);
    cudaFree(g.refs);
    cudaFree(g.stats_d);
    if (g.stats_h)
        cudaFreeHost(g.stats_h);
    cudaFree(g.sq);
    cudaFree(g.si);
    cudaFree(g.si2);
    cudaFree(g.jt);
    cudaFree(g.skey);
    cudaFree(g.qs);
    cudaFree(g.Lbuf);
    if (g.mb_h)
        cudaFreeHost(g.mb_h);
    cudaFree(g.hist);
    cudaFree(g.base);
    cudaFree(g.stage);
    for (auto &e : g.ev)
        if (e)
            cudaEventDestroy(e);
    for (int b = 0; b < 2; b++) {
        if (g.ev_done[b])
            cudaEventDestroy(g.ev_done[b]);
        if (g.ev_copied[b])
            cudaEventDestroy(g.ev_copied[b]);
    }
    if (g.copy_stream)
        cudaStreamDestroy(g.copy_stream);
}

uint64_t grid_checksum(const Grid &g)
{
    unsigned long long *d = nullptr;
    XS_CUDA_TRY(cudaMalloc(&d, sizeof(unsigned long long)));
    XS_CUDA_TRY(cudaMemset(d, 0, sizeof(unsigned long long)));
    uint64_t off = 0;
    auto add = [&](const void *p, int64_t bytes) {
        if (!p || bytes <= 0)
            return;
        const int64_t w = bytes / 4;
        k_checksum<<<grid_blocks(w, 256), 256>>>((const uint32_t *)p, w, off, d);
        off += (uint64_t)w;
    };
    add(g.E, g.N * 8);
    add(g.pts, g.N * 48);
    add(g.mats, 12 * (int64_t)g.max_nucs * 4);
    add(g.concs, 12 * (int64_t)g.max_nucs * 8);
    add(g.U, g.U ? g.N * 8 : 0);
    add(g.IDX, g.IDX ? g.N * g.n_nuc * 4 : 0);
    add(g.H, g.H ? g.bins * g.n_nuc * 4 : 0);
    unsigned long long h = 0;
    cudaError_t e = cudaMemcpy(&h, d, sizeof(h), cudaMemcpyDeviceToHost);
    cudaFree(d);
    XS_CUDA_TRY(e);
    return (uint64_t)h;
}

GridView make_view(const Grid &g)
{
    GridView v{};
    v.E = g.E;
    v.pts = g.pts;
    v.iv = g.iv;
    v.ivs = g.ivs;
    v.U = g.U;
    v.IDX = g.IDX;
    v.H = g.H;
    v.mats = g.mats;
    v.concs = g.concs;
    v.num_nucs = g.num_nucs_d;
    v.refs = (const NucRef *)g.refs;
    v.n = (int32_t)g.n;
    v.n_nuc = (int32_t)g.n_nuc;
    v.N = (int32_t)g.N;
    v.bins = (int32_t)g.bins;
    v.max_nucs = g.max_nucs;
    v.du = g.bins > 0 ? 1.0 / (double)g.bins : 0.0;
    v.tkeys = g.tkeys;
    v.t_levels = g.t_levels;
    for (int d = 0; d < kTreeMaxLevels; d++) {
        v.t_stride[d] = g.t_stride[d];
        v.t_off[d] = g.t_off[d];
    }
    v.t_leaf = g.t_leaf;
    v.t_per_nuc = (int32_t)g.t_per_nuc;
    v.b_log2 = g.bnd ? g.b_log2 : 0;
    v.bnd = g.bnd;
    v.u_log2 = g.ubnd ? g.u_log2 : 0;
    v.ubnd = g.ubnd;
    return v;
}

SampleView make_sample_view(const Grid &g, uint64_t seed, int64_t first, int64_t count)
{
    SampleView s{};
    s.seed = seed;
    s.first = first;
    s.count = count;
    for (int m = 0; m < 12; m++)
        s.T[m] = g.thresholds[m];
    return s;
}

} // namespace xs
