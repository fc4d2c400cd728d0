// lookup_fused.cu -- one thread per lookup, search + interpolation fused (XSBench's
// event kernel shape).  Used for XS_SORT_NONE (sampling fused in: the
// XSBench baseline order) and, with XS_FLAG_FUSED, for sorted lookups (the A/B against the
// split path of lookup_split.cu).
#include <algorithm>

#include "lookup_common.cuh"

namespace xs {

constexpr int kFusedTpb = 256;

template <int GRID, int SEARCH, bool SORTED>
__global__ void __launch_bounds__(kFusedTpb, 4)
    k_lookup(GridView gv, SampleView sv, SortedView so, Affine J_grid, double *__restrict__ out,
             int32_t *__restrict__ out_idx, unsigned long long *__restrict__ stats)
{
    __shared__ uint32_t s_mb[kMaterials + 1];
    if constexpr (SORTED) {
        if (threadIdx.x <= kMaterials)
            s_mb[threadIdx.x] = __ldg(so.mb_dev + threadIdx.x);
        __syncthreads();
    }
    uint32_t my_hash = 0, my_pairs = 0;
    const int count = (int)sv.count;
    const int G = gridDim.x * blockDim.x;
    int j = blockIdx.x * blockDim.x + threadIdx.x;
    uint64_t s = 0;
    uint32_t r_next = 0;
    double q_next = 0.0;
    if constexpr (!SORTED) {
        if (j < count)
            s = lookup_state(sv, j);
    } else if (j < count) {
        r_next = __ldg(so.slot + j);
        q_next = __ldg(so.q_of + r_next);
    }
    for (; j < count; j += G) {
        double q;
        int mat;
        uint32_t r;
        if constexpr (SORTED) {
            // the slot's lookup and energy were fetched one iteration ahead: the dependent
            // random 8 B read of q_of overlaps this lookup's ~15-300 nuclide searches
            q = q_next;
            r = r_next;
            if (j + G < count) {
                r_next = __ldg(so.slot + j + G);
                q_next = __ldg(so.q_of + r_next);
            }
            mat = material_of(s_mb, (uint32_t)j);
        } else {
            sample_lookup(s, sv, q, mat);
            r = (uint32_t)j;
            s = lcg_apply(J_grid, s);
        }
        const int nn = __ldg(gv.num_nucs + mat);
        const int row = mat * gv.max_nucs;
        const int e_union = union_index<GRID, SEARCH>(gv, q);
        Acc A;
        for (int jn = 0; jn < nn; jn++) {
            const int nuc = __ldg(gv.mats + row + jn);
            const double conc = __ldg(gv.concs + row + jn);
            const int L = lower_index<GRID, SEARCH>(gv, nuclide_row(gv, nuc), nuc, q, e_union);
            if (out_idx)
                out_idx[(size_t)r * gv.max_nucs + jn] = L;
            accumulate_pair(gv, nuc, L, q, conc, A);
        }
        my_hash += verify(A);
        my_pairs += (uint32_t)nn;
        if (out)
            store_macro(out, r, A);
    }
    reduce_stats<kFusedTpb>(my_hash, my_pairs, stats);
}

using FusedFn = void (*)(GridView, SampleView, SortedView, Affine, double *, int32_t *, unsigned long long *);

template <int GRID, int SEARCH> static FusedFn pick_s(bool sorted)
{
    return sorted ? k_lookup<GRID, SEARCH, true> : k_lookup<GRID, SEARCH, false>;
}

template <int GRID> static FusedFn pick_g(int search, bool sorted)
{
    switch (search) {
    case XS_SEARCH_M: return pick_s<GRID, XS_SEARCH_M>(sorted);
    case XS_SEARCH_U1: return pick_s<GRID, XS_SEARCH_U1>(sorted);
    case XS_SEARCH_U2: return pick_s<GRID, XS_SEARCH_U2>(sorted);
    case XS_SEARCH_U4: return pick_s<GRID, XS_SEARCH_U4>(sorted);
    case XS_SEARCH_U8: return pick_s<GRID, XS_SEARCH_U8>(sorted);
    case XS_SEARCH_B: return pick_s<GRID, XS_SEARCH_B>(sorted);
    case XS_SEARCH_M2: return pick_s<GRID, XS_SEARCH_M2>(sorted);
    case XS_SEARCH_M4: return pick_s<GRID, XS_SEARCH_M4>(sorted);
    default: return pick_s<GRID, XS_SEARCH_M8>(sorted);
    }
}

void launch_fused(int grid_type, int search, bool sorted, int blocks, int tpb, cudaStream_t stream,
                  const GridView &gv, const SampleView &sv, const SortedView &so, Affine J_grid, double *out,
                  int32_t *out_idx, unsigned long long *stats)
{
    FusedFn f = grid_type == XS_NUCLIDE     ? pick_g<XS_NUCLIDE>(search, sorted)
                : grid_type == XS_UNIONIZED ? pick_g<XS_UNIONIZED>(search, sorted)
                                            : pick_g<XS_HASH>(search, sorted);
    f<<<blocks, tpb, 0, stream>>>(gv, sv, so, J_grid, out, out_idx, stats);
    XS_CUDA_TRY(cudaGetLastError());
}

} // namespace xs
