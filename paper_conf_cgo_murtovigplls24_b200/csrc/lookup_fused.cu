// lookup_fused.cu -- one thread per lookup, search + interpolation fused (XSBench's
// event kernel shape).  Used for XS_SORT_NONE (sampling fused in: the
// XSBench baseline order) and, by default, for sorted lookups.
//
// The loop is warp-synchronous: each iteration a warp takes 32 consecutive lookup slots
// (lanes past the end idle), so warp collectives are legal inside it.  With XS_SEARCH_W
// on a nuclide grid, a warp whose 32 sorted lookups share one material searches each
// nuclide cooperatively (warp_bounds) and every lane finishes with Listing 1 inside the
// warp's window; any other warp runs the per-lane search.
#include <algorithm>

#include "lookup_common.cuh"

namespace xs {

constexpr int kFusedTpb = 256;
#ifndef XS_CHUNK_ITERS
#define XS_CHUNK_ITERS 4
#endif
constexpr int kChunkIters = XS_CHUNK_ITERS; // 256-slot iterations per work chunk (sorted)
#ifndef XS_WARP_QUEUE
#define XS_WARP_QUEUE 1
#endif
#ifndef XS_WARP_ITERS
#define XS_WARP_ITERS 4
#endif
// Sorted work queue granularity (measured): each warp pulls its own chunk
// of 4 x 32 slots (no CTA barrier, no waiting for the CTA's slowest warp): 1.03x (small) /
// 1.035x (large) over CTA chunks of 4 x 256; 2 x 32 and 8 x 32 are slower (large: 8 x 32
// widens the GPU's in-flight band past what L2 holds, 0.88x).
constexpr bool kWarpQueue = XS_WARP_QUEUE;
constexpr int kWarpIters = XS_WARP_ITERS;
#ifndef XS_W_MIN_BLOCKS
#define XS_W_MIN_BLOCKS 4
#endif
#ifndef XS_H_MIN_BLOCKS
#define XS_H_MIN_BLOCKS 4
#endif

// OUTS: the call asked for macroscopic XS and/or indices; without it the bench/hash path
// carries no output pointers (fewer live registers, no spills at 64 per thread).
// ILP2 (H on the nuclide grid only): two nuclides per iteration at 3 CTAs/SM -- chosen for
// long nuclide lists (large tables: 1.06x), where it beats the extra occupancy of ILP1
// (small tables: ILP1 is 1.05x faster).
template <int GRID, int SEARCH, bool SORTED, bool OUTS, bool ILP2 = false>
__global__ void __launch_bounds__(kFusedTpb, ILP2                    ? 3
                                             : SEARCH == XS_SEARCH_W ? XS_W_MIN_BLOCKS
                                             : SEARCH == XS_SEARCH_H ? XS_H_MIN_BLOCKS
                                                                     : 4)
    k_lookup(GridView gv, SampleView sv, SortedView so, Affine J_grid, double *__restrict__ out_,
             int32_t *__restrict__ out_idx_, unsigned long long *__restrict__ stats)
{
    double *__restrict__ out = OUTS ? out_ : nullptr;
    int32_t *__restrict__ out_idx = OUTS ? out_idx_ : nullptr;
    constexpr bool kCoop = SORTED && SEARCH == XS_SEARCH_W && GRID == XS_NUCLIDE;
#ifndef XS_PIPE_H // software-pipelined H path: measured slower (register spills) -> off
#define XS_PIPE_H 0
#endif
    constexpr bool kPipeH = XS_PIPE_H && SEARCH == XS_SEARCH_H && GRID == XS_NUCLIDE;
    constexpr bool kIlp2 = ILP2 && SEARCH == XS_SEARCH_H && GRID == XS_NUCLIDE;
    __shared__ uint32_t s_mb[kMaterials + 1];
    if constexpr (SORTED) {
        if (threadIdx.x <= kMaterials)
            s_mb[threadIdx.x] = __ldg(so.mb_dev + threadIdx.x);
        __syncthreads();
    }
    uint32_t my_hash = 0, my_pairs = 0;
    const int lane = threadIdx.x & 31;
    const int count = (int)sv.count;
    // Sorted: a persistent grid pulls chunks of kChunkIters x blockDim consecutive slots
    // from an atomic counter, in slot order: consecutive iterations of a CTA hit
    // neighbouring grid intervals (L1 reuse), the whole GPU sweeps the sorted order as one
    // narrow band (L2 reuse when the grid does not fit), and the load balances itself.
    // Unsorted: grid-stride over the chunk (XSBench order).
    __shared__ int s_chunk;
    const int csize = !SORTED ? 0 : kWarpQueue ? kWarpIters * 32 : kChunkIters * (int)blockDim.x;
    const int tpos = kWarpQueue ? lane : (int)threadIdx.x; // position inside a chunk
    int j0, jend, G;
    if constexpr (SORTED) {
        int c;
        if constexpr (kWarpQueue) {
            if (lane == 0)
                c = atomicAdd(so.work, 1);
            c = __shfl_sync(0xffffffffu, c, 0);
        } else {
            if (threadIdx.x == 0)
                s_chunk = atomicAdd(so.work, 1);
            __syncthreads();
            c = s_chunk;
        }
        j0 = c * csize + tpos;
        jend = min(count, c * csize + csize);
        G = kWarpQueue ? 32 : blockDim.x;
    } else {
        j0 = blockIdx.x * blockDim.x + threadIdx.x;
        jend = count;
        G = gridDim.x * blockDim.x;
    }
    uint64_t s = 0;
    uint32_t r_next = 0;
    double q_next = 0.0;
    const uint64_t pol = policy_evict_first();
    if constexpr (!SORTED) {
        if (j0 < count)
            s = lookup_state(sv, j0);
    }
    for (;;) {
        if constexpr (SORTED) {
            if (j0 - tpos >= count)
                break;
            if (j0 < jend) {
                r_next = ld_stream(so.slot + j0, pol);
                q_next = so.q ? ld_stream(so.q + j0, pol) : ld_stream(so.q_of + r_next, pol);
            }
        }
    for (int jw = j0 - lane; jw < jend; jw += G) { // warp-uniform trip count
        const int j = jw + lane;
        const bool active = j < jend;
        double q = 0.0;
        int mat = 0;
        uint32_t r = 0;
        if (active) {
            if constexpr (SORTED) {
                // this slot's lookup and energy were fetched one iteration ahead: the
                // dependent random 8 B read of q_of overlaps a whole lookup's searches
                q = q_next;
                r = r_next;
                if (j + G < jend) {
                    r_next = ld_stream(so.slot + j + G, pol);
                    q_next = so.q ? ld_stream(so.q + j + G, pol) : ld_stream(so.q_of + r_next, pol);
                }
                mat = material_of(s_mb, (uint32_t)j);
            } else {
                sample_lookup(s, sv, q, mat);
                r = (uint32_t)j;
                s = lcg_apply(J_grid, s);
            }
        }
        const int nn = active ? __ldg(gv.num_nucs + mat) : 0;
        const int row = mat * gv.max_nucs;
        Acc A;
        bool coop = false;
        if constexpr (kCoop) {
            const int mat0 = __shfl_sync(0xffffffffu, mat, 0);
            coop = __all_sync(0xffffffffu, active && mat == mat0) && tree_usable(gv);
        }
        if (coop) { // warp-uniform branch: all 32 lanes, same material, same nuclides
            const double q_lo = warp_min(q), q_hi = warp_max(q);
            for (int jn = 0; jn < nn; jn++) {
                const Row rw = load_row(gv, row + jn);
                int L_lo, L_hi;
                warp_bounds(gv, rw.E, rw.T, q_lo, q_hi, L_lo, L_hi);
                const int L = (L_lo == L_hi) ? L_lo : search<XS_SEARCH_U2>(rw.E, L_lo, L_hi + 1, q);
                if (out_idx)
                    out_idx[(size_t)r * gv.max_nucs + jn] = L;
                accumulate_pair(rw.pts, L, q, rw.conc, A);
            }
        } else if (kIlp2 && active) {
            // bin-bounded search, two nuclides per iteration: both rows, bins and 96 B
            // gathers are independent, so their latency chains overlap; the accumulation
            // stays in ascending nuclide order (reading R8), bit-identical to one at a time
            const bool in01 = q >= 0.0 && q <= 1.0 && gv.b_log2 > 0;
            const int bq = in01 ? bin_of(q, gv.b_log2) : 0;
            const Bin full{0, gv.n - 2, 0.0};
            int jn = 0;
            for (; jn + 1 < nn; jn += 2) {
                const Row ra = load_row(gv, row + jn), rb = load_row(gv, row + jn + 1);
                const Bin ba = in01 ? load_bin(ra.B + bq) : full;
                const Bin bb = in01 ? load_bin(rb.B + bq) : full;
                const int La = bin_lower(ra.E, ba, q), Lb = bin_lower(rb.E, bb, q);
                if (out_idx) {
                    out_idx[(size_t)r * gv.max_nucs + jn] = La;
                    out_idx[(size_t)r * gv.max_nucs + jn + 1] = Lb;
                }
                accumulate_pair2(ra.pts, La, ra.conc, rb.pts, Lb, rb.conc, q, A);
            }
            if (jn < nn) {
                const Row ra = load_row(gv, row + jn);
                const int La = bin_lower(ra.E, in01 ? load_bin(ra.B + bq) : full, q);
                if (out_idx)
                    out_idx[(size_t)r * gv.max_nucs + jn] = La;
                accumulate_pair(ra.pts, La, q, ra.conc, A);
            }
        } else if (kPipeH && active) {
            // bin-bounded search, software-pipelined: the next nuclide's row and bin entry
            // (independent of this nuclide) load while this one is resolved, gathered and
            // interpolated
            const bool in01 = q >= 0.0 && q <= 1.0 && gv.b_log2 > 0;
            const int bq = in01 ? bin_of(q, gv.b_log2) : 0;
            const Bin full{0, gv.n - 2, 0.0}; // window [0, n-1]: the full search
            Row rw = load_row(gv, row);
            Bin bn = in01 ? load_bin(rw.B + bq) : full;
            for (int jn = 0; jn < nn; jn++) {
                Row rn = rw;
                Bin bn_n = bn;
                if (jn + 1 < nn) {
                    rn = load_row(gv, row + jn + 1);
                    bn_n = in01 ? load_bin(rn.B + bq) : full;
                }
                const int L = bin_lower(rw.E, bn, q);
                if (out_idx)
                    out_idx[(size_t)r * gv.max_nucs + jn] = L;
                accumulate_pair(rw.pts, L, q, rw.conc, A);
                rw = rn;
                bn = bn_n;
            }
        } else if (active) {
            const int e_union = union_index<GRID, SEARCH>(gv, q);
            for (int jn = 0; jn < nn; jn++) {
                const Row rw = load_row(gv, row + jn);
                const int L = lower_index<GRID, SEARCH>(gv, rw, q, e_union);
                if (out_idx)
                    out_idx[(size_t)r * gv.max_nucs + jn] = L;
                accumulate_pair(rw.pts, L, q, rw.conc, A);
            }
        }
        if (active) {
            my_hash += verify(A);
            my_pairs += (uint32_t)nn;
            if (out)
                store_macro(out, r, A);
        }
    }
        if constexpr (!SORTED)
            break;
        else { // next chunk
            int c;
            if constexpr (kWarpQueue) {
                if (lane == 0)
                    c = atomicAdd(so.work, 1);
                c = __shfl_sync(0xffffffffu, c, 0);
            } else {
                __syncthreads();
                if (threadIdx.x == 0)
                    s_chunk = atomicAdd(so.work, 1);
                __syncthreads();
                c = s_chunk;
            }
            j0 = c * csize + tpos;
            jend = min(count, c * csize + csize);
        }
    }
    reduce_stats<kFusedTpb>(my_hash, my_pairs, stats);
}

// XSBench history order: thread p runs particle p's `hl` lookups one after the other, its
// stream continuing (two draws per lookup: the 2-step affine map); lookup i of the range
// is particle i / hl, step i % hl, so results equal the event order's exactly
template <int GRID, int SEARCH, bool OUTS>
__global__ void __launch_bounds__(kFusedTpb, 4)
    k_history(GridView gv, SampleView sv, int hl, Affine J2, double *__restrict__ out_, int32_t *__restrict__ out_idx_,
              unsigned long long *__restrict__ stats)
{
    double *__restrict__ out = OUTS ? out_ : nullptr;
    int32_t *__restrict__ out_idx = OUTS ? out_idx_ : nullptr;
    uint32_t my_hash = 0, my_pairs = 0;
    const int64_t count = sv.count;
    const int64_t particles = (count + hl - 1) / hl;
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < particles;
         p += (int64_t)gridDim.x * blockDim.x) {
        uint64_t s = lookup_state(sv, p * hl); // Listing-7 jump once per particle
        const int64_t i_end = min(count, (p + 1) * hl);
        for (int64_t i = p * hl; i < i_end; i++) {
            double q;
            int mat;
            sample_lookup(s, sv, q, mat);
            s = lcg_apply(J2, s);
            const int nn = __ldg(gv.num_nucs + mat);
            const int row = mat * gv.max_nucs;
            const int e_union = union_index<GRID, SEARCH>(gv, q);
            Acc A;
            for (int jn = 0; jn < nn; jn++) {
                const Row rw = load_row(gv, row + jn);
                const int L = lower_index<GRID, SEARCH>(gv, rw, q, e_union);
                if (out_idx)
                    out_idx[(size_t)i * gv.max_nucs + jn] = L;
                accumulate_pair(rw.pts, L, q, rw.conc, A);
            }
            my_hash += verify(A);
            my_pairs += (uint32_t)nn;
            if (out)
                store_macro(out, (uint32_t)i, A);
        }
    }
    reduce_stats<kFusedTpb>(my_hash, my_pairs, stats);
}

using HistFn = void (*)(GridView, SampleView, int, Affine, double *, int32_t *, unsigned long long *);

template <int GRID> static HistFn pick_hist_g(int search, bool outs)
{
#define XS_HIST_CASE(S)                                                                                      \
    case S: return outs ? k_history<GRID, S, true> : k_history<GRID, S, false>;
    switch (search) {
        XS_HIST_CASE(XS_SEARCH_M)
        XS_HIST_CASE(XS_SEARCH_U1)
        XS_HIST_CASE(XS_SEARCH_U2)
        XS_HIST_CASE(XS_SEARCH_U4)
        XS_HIST_CASE(XS_SEARCH_U8)
        XS_HIST_CASE(XS_SEARCH_B)
        XS_HIST_CASE(XS_SEARCH_M2)
        XS_HIST_CASE(XS_SEARCH_M4)
        XS_HIST_CASE(XS_SEARCH_M8)
        XS_HIST_CASE(XS_SEARCH_W)
    default: return outs ? k_history<GRID, XS_SEARCH_H, true> : k_history<GRID, XS_SEARCH_H, false>;
    }
#undef XS_HIST_CASE
}

void launch_history(int grid_type, int search, int hl, int blocks, cudaStream_t stream, const GridView &gv,
                    const SampleView &sv, double *out, int32_t *out_idx, unsigned long long *stats)
{
    const bool outs = out || out_idx;
    HistFn f = grid_type == XS_NUCLIDE     ? pick_hist_g<XS_NUCLIDE>(search, outs)
               : grid_type == XS_UNIONIZED ? pick_hist_g<XS_UNIONIZED>(search, outs)
                                           : pick_hist_g<XS_HASH>(search, outs);
    f<<<blocks, kFusedTpb, 0, stream>>>(gv, sv, hl, lcg_jump(2), out, out_idx, stats);
    XS_CUDA_TRY(cudaGetLastError());
}

using FusedFn = void (*)(GridView, SampleView, SortedView, Affine, double *, int32_t *, unsigned long long *);

template <int GRID, int SEARCH> static FusedFn pick_s(bool sorted, bool outs)
{
    if (sorted)
        return outs ? k_lookup<GRID, SEARCH, true, true> : k_lookup<GRID, SEARCH, true, false>;
    return outs ? k_lookup<GRID, SEARCH, false, true> : k_lookup<GRID, SEARCH, false, false>;
}

template <int GRID> static FusedFn pick_g(int search, bool sorted, bool outs)
{
    switch (search) {
    case XS_SEARCH_M: return pick_s<GRID, XS_SEARCH_M>(sorted, outs);
    case XS_SEARCH_U1: return pick_s<GRID, XS_SEARCH_U1>(sorted, outs);
    case XS_SEARCH_U2: return pick_s<GRID, XS_SEARCH_U2>(sorted, outs);
    case XS_SEARCH_U4: return pick_s<GRID, XS_SEARCH_U4>(sorted, outs);
    case XS_SEARCH_U8: return pick_s<GRID, XS_SEARCH_U8>(sorted, outs);
    case XS_SEARCH_B: return pick_s<GRID, XS_SEARCH_B>(sorted, outs);
    case XS_SEARCH_M2: return pick_s<GRID, XS_SEARCH_M2>(sorted, outs);
    case XS_SEARCH_M4: return pick_s<GRID, XS_SEARCH_M4>(sorted, outs);
    case XS_SEARCH_M8: return pick_s<GRID, XS_SEARCH_M8>(sorted, outs);
    case XS_SEARCH_W: return pick_s<GRID, XS_SEARCH_W>(sorted, outs);
    default: return pick_s<GRID, XS_SEARCH_H>(sorted, outs);
    }
}

void launch_fused(int grid_type, int search, bool sorted, int blocks, int tpb, cudaStream_t stream,
                  const GridView &gv, const SampleView &sv, const SortedView &so, Affine J_grid, double *out,
                  int32_t *out_idx, unsigned long long *stats)
{
    const bool outs = out || out_idx;
    FusedFn f = grid_type == XS_NUCLIDE     ? pick_g<XS_NUCLIDE>(search, sorted, outs)
                : grid_type == XS_UNIONIZED ? pick_g<XS_UNIONIZED>(search, sorted, outs)
                                            : pick_g<XS_HASH>(search, sorted, outs);
    if (grid_type == XS_NUCLIDE && search == XS_SEARCH_H && sorted && gv.max_nucs > 64) {
        f = outs ? k_lookup<XS_NUCLIDE, XS_SEARCH_H, true, true, true>
                 : k_lookup<XS_NUCLIDE, XS_SEARCH_H, true, false, true>;
        blocks = std::min(blocks, blocks / 4 * 3 > 0 ? blocks / 4 * 3 : blocks); // one wave at 3 CTAs/SM
    }
    if (search == XS_SEARCH_S && sorted) { // the staged-window kernel (lookup_staged.cu)
        launch_staged(grid_type, blocks, tpb, stream, gv, sv, so, out, out_idx, stats);
        return;
    }
    f<<<blocks, tpb, 0, stream>>>(gv, sv, so, J_grid, out, out_idx, stats);
    XS_CUDA_TRY(cudaGetLastError());
}

} // namespace xs
