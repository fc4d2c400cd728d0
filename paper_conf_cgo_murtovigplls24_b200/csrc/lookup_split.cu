// lookup_split.cu -- the sorted hot path as two kernels.
//
//   k_search  every (lookup, nuclide) pair's lower index L into the pair buffer.  Only
//             the paper's loop runs here (Listing 1 in the chosen variant), with ~30
//             registers per thread so 64 warps per SM keep 64 dependent probe chains in
//             flight -- the chain latency, not bandwidth, bounds this kernel.
//   k_interp  per lookup: for each nuclide read L (coalesced), gather the two 48 B point
//             records, interpolate the 5 channels and accumulate density-weighted in
//             ascending nuclide order (reading R8); argmax; fused (hash, pairs) epilogue.
// The pair buffer is nuclide-major inside each material ([jn][j - matbase[m]]), so both
// kernels' warps store and load 32 consecutive int32 (one 128 B line) per nuclide.
#include <algorithm>

#include "lookup_common.cuh"

namespace xs {

// SortedView / PairView tables indexed by the (runtime) material: staged in shared
// memory so they are not copied to the local-memory stack frame.
struct MatTables {
    uint32_t mb[kMaterials + 1];
    uint64_t pb[kMaterials];
};

__device__ __forceinline__ void stage_tables(MatTables &t, const SortedView &so, const PairView &pv)
{
    if (threadIdx.x == 0) { // constant indices: read straight from the parameter bank
#pragma unroll
        for (int m = 0; m <= kMaterials; m++)
            t.mb[m] = so.matbase[m];
#pragma unroll
        for (int m = 0; m < kMaterials; m++)
            t.pb[m] = pv.pairbase[m];
    }
    __syncthreads();
}

template <int GRID, int SEARCH>
__global__ void __launch_bounds__(kSearchTpb, 8)
    k_search(GridView gv, SortedView so, PairView pv)
{
    __shared__ MatTables t;
    stage_tables(t, so, pv);
    const uint32_t count = t.mb[kMaterials];
    for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < count; j += gridDim.x * blockDim.x) {
        const double q = so.q[j];
        const int mat = material_of(t.mb, j);
        const uint32_t local = j - t.mb[mat];
        const uint32_t stride = t.mb[mat + 1] - t.mb[mat];
        int32_t *__restrict__ dst = pv.L + t.pb[mat] + local;
        const int nn = __ldg(gv.num_nucs + mat);
        const int row = mat * gv.max_nucs;
        const int e_union = union_index<GRID, SEARCH>(gv, q);
        for (int jn = 0; jn < nn; jn++) {
            const Row rw = load_row(gv, row + jn);
            dst[(size_t)jn * stride] = lower_index<GRID, SEARCH>(gv, rw, q, e_union);
        }
    }
}

__global__ void __launch_bounds__(kInterpTpb, 2)
    k_interp(GridView gv, SortedView so, PairView pv, double *__restrict__ out, int32_t *__restrict__ out_idx,
             unsigned long long *__restrict__ stats)
{
    __shared__ MatTables t;
    stage_tables(t, so, pv);
    uint32_t my_hash = 0, my_pairs = 0;
    const uint32_t count = t.mb[kMaterials];
    for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < count; j += gridDim.x * blockDim.x) {
        const double q = so.q[j];
        const int mat = material_of(t.mb, j);
        const uint32_t local = j - t.mb[mat];
        const uint32_t stride = t.mb[mat + 1] - t.mb[mat];
        const int32_t *__restrict__ src = pv.L + t.pb[mat] + local;
        const int nn = __ldg(gv.num_nucs + mat);
        const int row = mat * gv.max_nucs;
        const uint32_t r = (out || out_idx) ? so.slot[j] : 0u;
        Acc A;
        for (int jn = 0; jn < nn; jn++) {
            const Row rw = load_row(gv, row + jn);
            const int L = __ldg(src + (size_t)jn * stride);
            if (out_idx)
                out_idx[(size_t)r * gv.max_nucs + jn] = L;
            accumulate_pair(rw.pts, L, q, rw.conc, A);
        }
        my_hash += verify(A);
        my_pairs += (uint32_t)nn;
        if (out)
            store_macro(out, r, A);
    }
    reduce_stats<kInterpTpb>(my_hash, my_pairs, stats);
}

using SearchKFn = void (*)(GridView, SortedView, PairView);

template <int GRID> static SearchKFn pick_g(int search)
{
    switch (search) {
    case XS_SEARCH_M: return k_search<GRID, XS_SEARCH_M>;
    case XS_SEARCH_U1: return k_search<GRID, XS_SEARCH_U1>;
    case XS_SEARCH_U2: return k_search<GRID, XS_SEARCH_U2>;
    case XS_SEARCH_U4: return k_search<GRID, XS_SEARCH_U4>;
    case XS_SEARCH_U8: return k_search<GRID, XS_SEARCH_U8>;
    case XS_SEARCH_B: return k_search<GRID, XS_SEARCH_B>;
    case XS_SEARCH_M2: return k_search<GRID, XS_SEARCH_M2>;
    case XS_SEARCH_M4: return k_search<GRID, XS_SEARCH_M4>;
    case XS_SEARCH_M8: return k_search<GRID, XS_SEARCH_M8>;
    case XS_SEARCH_W: return k_search<GRID, XS_SEARCH_W>;
    default: return k_search<GRID, XS_SEARCH_H>;
    }
}

void launch_search(int grid_type, int search, int blocks, cudaStream_t stream, const GridView &gv,
                   const SortedView &so, const PairView &pv)
{
    SearchKFn f = grid_type == XS_NUCLIDE     ? pick_g<XS_NUCLIDE>(search)
                  : grid_type == XS_UNIONIZED ? pick_g<XS_UNIONIZED>(search)
                                              : pick_g<XS_HASH>(search);
    f<<<blocks, kSearchTpb, 0, stream>>>(gv, so, pv);
    XS_CUDA_TRY(cudaGetLastError());
}

void launch_interp(int blocks, cudaStream_t stream, const GridView &gv, const SortedView &so, const PairView &pv,
                   double *out, int32_t *out_idx, unsigned long long *stats)
{
    k_interp<<<blocks, kInterpTpb, 0, stream>>>(gv, so, pv, out, out_idx, stats);
    XS_CUDA_TRY(cudaGetLastError());
}

} // namespace xs
