// lookup_common.cuh -- device pieces shared by the lookup kernels.
#pragma once
#include "search.cuh"
#include "xs_internal.cuh"

namespace xs {

// ---- sampling ------------------------------------------------
// `s` is skip(seed, 2i): q is the draw at stream position 2i, the pick_mat roll at 2i+1.
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

// skip(seed, 2*(first + j)) with the Listing-7 loop (kept merged: PAPER.md:474)
__device__ __forceinline__ uint64_t lookup_state(const SampleView &sv, int64_t j)
{
    return lcg_apply(lcg_jump(2 * (uint64_t)(sv.first + j)), sv.seed);
}

// Sort buckets: material m owns keys [kbase[m], kbase[m] + nb[m]), nb[m] proportional to
// its expected share of (lookup, nuclide) pairs, so the material that dominates the cost
// gets the finest energy resolution.  Any key assignment is a valid ordering.
struct BucketPlan {
    int K;
    int nb[kMaterials];
    int kbase[kMaterials + 1];
};

// nb / kbase are read from shared memory: indexed by a per-lane material, a parameter-bank
// read would serialise over the distinct materials of the warp
__device__ __forceinline__ int bucket_key(const int *s_nb, const int *s_kbase, int mat, double q)
{
    const int nb = s_nb[mat];
    const int b = (int)__dmul_rn(q, (double)nb);
    return s_kbase[mat] + (b < nb - 1 ? b : nb - 1); // q may be exactly 1.0 (R7)
}

// material of sorted position j: the number of later materials whose first slot is <= j
__device__ __forceinline__ int material_of(const uint32_t *mb, uint32_t j)
{
    int mat = 0;
#pragma unroll
    for (int m = 1; m < kMaterials; m++)
        mat += (j >= mb[m]) ? 1 : 0;
    return mat;
}

// ---- streaming loads: read once, keep them from evicting the grid out of L2 ----------------
__device__ __forceinline__ uint64_t policy_evict_first()
{
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

__device__ __forceinline__ uint32_t ld_stream(const uint32_t *a, uint64_t pol)
{
    uint32_t v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
    return v;
}

__device__ __forceinline__ double ld_stream(const double *a, uint64_t pol)
{
    double v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(a), "l"(pol));
    return v;
}

// ---- nuclide j of material m --------------------------------------------------------------
struct Row {
    const double *E, *pts, *T;
    const BinEntry *B;
    double conc;
    int nuc;
};

struct Bin {
    int lo, cnt;
    double e_next;
};

__device__ __forceinline__ Bin load_bin(const BinEntry *p)
{
    const int4 v = __ldg(reinterpret_cast<const int4 *>(p));
    return Bin{v.x, v.y, __hiloint2double(v.w, v.z)};
}

// the bin of q: q * 2^k is exact, so b/2^k <= q < (b+1)/2^k (q = 1.0 -> last bin)
__device__ __forceinline__ int bin_of(double q, int log2_bins)
{
    const int nb = 1 << log2_bins;
    const int b = (int)__dmul_rn(q, (double)nb);
    return b < nb - 1 ? b : nb - 1;
}

// L(q) from its bin: no row access when the bin holds <= 1 point, else Listing 1 on the
// bin's window [lo, lo + cnt + 1] (L monotone: lo <= L(q) <= lo + cnt <= n-2)
__device__ __forceinline__ int bin_lower(const double *__restrict__ A, const Bin &bn, double q)
{
    if (bn.cnt <= 1)
        return bn.lo + ((bn.cnt == 1 && bn.e_next <= q) ? 1 : 0);
    return kBinK4 ? search_K4(A, bn.lo, bn.lo + bn.cnt + 1, q) : search<XS_SEARCH_U2>(A, bn.lo, bn.lo + bn.cnt + 1, q);
}

// 48 B NucRef as three 16 B broadcast loads (fields a kernel does not use are dead code)
__device__ __forceinline__ Row load_row(const GridView &gv, int idx)
{
    const ulonglong2 *p = reinterpret_cast<const ulonglong2 *>(gv.refs + idx);
    const ulonglong2 a = __ldg(p), b = __ldg(p + 1), c = __ldg(p + 2);
    Row r;
    r.E = opaque(reinterpret_cast<const double *>(a.x));
    r.pts = opaque(reinterpret_cast<const double *>(a.y));
    r.T = opaque(reinterpret_cast<const double *>(b.x));
    r.B = reinterpret_cast<const BinEntry *>(b.y);
    r.conc = __longlong_as_double((long long)c.x);
    r.nuc = (int)c.y;
    return r;
}

// the Row of nuclide `nuc` built from the grid view (debug paths that have no material)
__device__ __forceinline__ Row make_row(const GridView &gv, int nuc)
{
    Row r;
    r.E = opaque(gv.E + (size_t)nuc * (uint32_t)gv.n);
    r.pts = kIv ? gv.iv + (size_t)nuc * (uint32_t)(gv.n - 1) * 12 : gv.pts + (size_t)nuc * (uint32_t)gv.n * 6;
    r.T = gv.tkeys ? gv.tkeys + (size_t)nuc * (uint32_t)gv.t_per_nuc : nullptr;
    r.B = gv.bnd ? gv.bnd + ((size_t)nuc << gv.b_log2) : nullptr;
    r.conc = 0.0;
    r.nuc = nuc;
    return r;
}

// ---- the lower index of one (lookup, nuclide) pair ----------------------
template <int GRID, int SEARCH>
__device__ __forceinline__ int lower_index(const GridView &gv, const Row &rw, double q, int e_union)
{
    const double *__restrict__ Ei = rw.E;
    const int nuc = rw.nuc;
    if constexpr (GRID == XS_NUCLIDE && (SEARCH == XS_SEARCH_H || SEARCH == XS_SEARCH_S)) {
        // bin-bounded window
        if (gv.b_log2 > 0 && q >= 0.0 && q <= 1.0)
            return bin_lower(Ei, load_bin(rw.B + bin_of(q, gv.b_log2)), q);
        return search<XS_SEARCH_U2>(Ei, 0, gv.n - 1, q);
    } else if constexpr (GRID == XS_NUCLIDE) {
        return search<SEARCH>(Ei, 0, gv.n - 1, q);
    } else if constexpr (GRID == XS_UNIONIZED) {
        return __ldg(gv.IDX + (size_t)e_union * (uint32_t)gv.n_nuc + nuc);
    } else if constexpr (kHashFast && (SEARCH == XS_SEARCH_H || SEARCH == XS_SEARCH_S)) {
        // R7's window by a shorter dependent chain (H and S only; the paper's variants keep
        // R7 as written).  Any bin b in range gives L(q) exactly: Listing 1 on [lo, hi] returns
        // L(q) whenever E[lo] <= q < E[hi] (or hi = n-1), and the guards send every other q to
        // the full search -- so b comes from a multiply instead of the IEEE division (they
        // differ only where RN(q bins) and RN(q / du) straddle an integer), and the two guard
        // energies are loaded alongside the window search instead of before it.
        int64_t b = (int64_t)__dmul_rn(q, (double)gv.bins);
        b = b < 0 ? 0 : (b > gv.bins - 1 ? gv.bins - 1 : b);
        const int lo = __ldg(gv.H + b * gv.n_nuc + nuc);
        const int hi = (b == gv.bins - 1) ? gv.n - 1 : __ldg(gv.H + (b + 1) * gv.n_nuc + nuc) + 1;
        const double e_lo = __ldg(Ei + lo), e_hi = __ldg(Ei + hi);
        int L = kHashK4 ? search_K4(Ei, lo, hi, q) : search<SEARCH>(Ei, lo, hi, q);
        if (q < e_lo || (hi < gv.n - 1 && q >= e_hi))
            L = search<SEARCH>(Ei, 0, gv.n - 1, q);
        return L;
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
    if constexpr (GRID == XS_UNIONIZED && (SEARCH == XS_SEARCH_H || SEARCH == XS_SEARCH_S)) {
        // the same bin-bounded window over the unionized energies (R4 + §6.5)
        if (gv.u_log2 > 0 && q >= 0.0 && q <= 1.0)
            return bin_lower(opaque(gv.U), load_bin(gv.ubnd + bin_of(q, gv.u_log2)), q);
        return search<XS_SEARCH_U2>(opaque(gv.U), 0, gv.N - 1, q);
    } else if constexpr (GRID == XS_UNIONIZED) {
        return search<SEARCH>(opaque(gv.U), 0, gv.N - 1, q);
    } else {
        return 0;
    }
}

__device__ __forceinline__ const double *nuclide_row(const GridView &gv, int nuc)
{
    return opaque(gv.E + (size_t)nuc * (uint32_t)gv.n);
}

// ---- warp-cooperative bounds (XS_SEARCH_W) ----------------------------------
// All 32 lanes of a warp whose lookups share a material call this for the same nuclide.
// Lanes 0-15 find ub(q_lo) and lanes 16-31 ub(q_hi), ub(q) = #{k : E[k] <= q}: at each
// level a half-warp loads one 16-key node (one 128 B line) of the separator tree, counts
// the keys <= its query with one ballot, and descends into child c; the leaf compares
// <= 16 consecutive energies.  Returns L(q_lo), L(q_hi) = clamp(ub - 1, 0, n-2) in every
// lane, so each lane's L(q) lies in [L_lo, L_hi] (q_lo <= q <= q_hi, L monotone).
__device__ __forceinline__ bool tree_usable(const GridView &gv) { return gv.tkeys != nullptr || gv.n <= kTreeFan; }

__device__ __forceinline__ void warp_bounds(const GridView &gv, const double *__restrict__ Ei,
                                            const double *__restrict__ T, double q_lo, double q_hi, int &L_lo,
                                            int &L_hi)
{
    const int lane = threadIdx.x & 31, t = lane & 15;
    const double qh = lane < 16 ? q_lo : q_hi;
    const unsigned half = lane < 16 ? 0x0000FFFFu : 0xFFFF0000u;
    int base = 0, node = 0;
#pragma unroll
    for (int d = 0; d < kTreeMaxLevels; d++) {
        if (d < gv.t_levels) {
            const double key = __ldg(T + (uint32_t)(gv.t_off[d] + node * kTreeFan + t));
            const int c = __popc(__ballot_sync(0xffffffffu, key <= qh) & half);
            base += c * gv.t_stride[d];
            node = node * 17 + c;
        }
    }
    const int pos = base + t;
    const double key = (t < gv.t_leaf && pos < gv.n) ? __ldg(Ei + (uint32_t)pos)
                                                     : __longlong_as_double(0x7FF0000000000000ll);
    const int ub = base + __popc(__ballot_sync(0xffffffffu, key <= qh) & half);
    const int ub_lo = __shfl_sync(0xffffffffu, ub, 0);
    const int ub_hi = __shfl_sync(0xffffffffu, ub, 16);
    L_lo = min(max(ub_lo - 1, 0), gv.n - 2);
    L_hi = min(max(ub_hi - 1, 0), gv.n - 2);
}

__device__ __forceinline__ double warp_min(double v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
        v = fmin(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

__device__ __forceinline__ double warp_max(double v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
        v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// ---- interpolation + accumulation of one pair (reading R8) ------------------------------
struct Acc {
    double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0, a4 = 0.0;
};

// The interpolation of one pair (reading R8): f = (E_hi - q) / (E_hi - E_lo) by IEEE
// division, micro_c = fma(-f, X_hi - X_lo, X_hi), acc_c = fma(micro_c, conc, acc_c).
#if XS_IV
// 96 B gather of interval L's record {E_hi, dE, (X_hi, dX) x 5}: six 16 B loads; dE and dX
// were rounded at build time exactly as below, so the results are bit-identical
__device__ __forceinline__ void accumulate_pair(const double *__restrict__ iv_row, int L, double q, double conc,
                                                Acc &A)
{
    const double2 *p = reinterpret_cast<const double2 *>(iv_row) + (uint32_t)L * 6;
    const double2 e = __ldg(p + 0), c0 = __ldg(p + 1), c1 = __ldg(p + 2);
    const double2 c2 = __ldg(p + 3), c3 = __ldg(p + 4), c4 = __ldg(p + 5);
    const double f = __ddiv_rn(__dsub_rn(e.x, q), e.y);
    A.a0 = __fma_rn(__fma_rn(-f, c0.y, c0.x), conc, A.a0);
    A.a1 = __fma_rn(__fma_rn(-f, c1.y, c1.x), conc, A.a1);
    A.a2 = __fma_rn(__fma_rn(-f, c2.y, c2.x), conc, A.a2);
    A.a3 = __fma_rn(__fma_rn(-f, c3.y, c3.x), conc, A.a3);
    A.a4 = __fma_rn(__fma_rn(-f, c4.y, c4.x), conc, A.a4);
}

__device__ __forceinline__ void accumulate_pair2(const double *__restrict__ pa, int La, double ca,
                                                 const double *__restrict__ pb, int Lb, double cb, double q, Acc &A)
{
    const double2 *p = reinterpret_cast<const double2 *>(pa) + (uint32_t)La * 6;
    const double2 *s = reinterpret_cast<const double2 *>(pb) + (uint32_t)Lb * 6;
    const double2 e = __ldg(p + 0), c0 = __ldg(p + 1), c1 = __ldg(p + 2);
    const double2 c2 = __ldg(p + 3), c3 = __ldg(p + 4), c4 = __ldg(p + 5);
    const double2 g = __ldg(s + 0), d0 = __ldg(s + 1), d1 = __ldg(s + 2);
    const double2 d2 = __ldg(s + 3), d3 = __ldg(s + 4), d4 = __ldg(s + 5);
    const double fa = __ddiv_rn(__dsub_rn(e.x, q), e.y);
    const double fb = __ddiv_rn(__dsub_rn(g.x, q), g.y);
    const double a0 = __fma_rn(-fa, c0.y, c0.x), b0 = __fma_rn(-fb, d0.y, d0.x);
    const double a1 = __fma_rn(-fa, c1.y, c1.x), b1 = __fma_rn(-fb, d1.y, d1.x);
    const double a2 = __fma_rn(-fa, c2.y, c2.x), b2 = __fma_rn(-fb, d2.y, d2.x);
    const double a3 = __fma_rn(-fa, c3.y, c3.x), b3 = __fma_rn(-fb, d3.y, d3.x);
    const double a4 = __fma_rn(-fa, c4.y, c4.x), b4 = __fma_rn(-fb, d4.y, d4.x);
    A.a0 = __fma_rn(b0, cb, __fma_rn(a0, ca, A.a0));
    A.a1 = __fma_rn(b1, cb, __fma_rn(a1, ca, A.a1));
    A.a2 = __fma_rn(b2, cb, __fma_rn(a2, ca, A.a2));
    A.a3 = __fma_rn(b3, cb, __fma_rn(a3, ca, A.a3));
    A.a4 = __fma_rn(b4, cb, __fma_rn(a4, ca, A.a4));
}
#else
// 96 B gather: the 48 B records of points L and L+1, three 16 B loads each
__device__ __forceinline__ void accumulate_pair(const double *__restrict__ pts_row, int L, double q, double conc,
                                                Acc &A)
{
    const double2 *p = reinterpret_cast<const double2 *>(pts_row) + (uint32_t)L * 3;
    const double2 l0 = __ldg(p + 0), l1 = __ldg(p + 1), l2 = __ldg(p + 2);
    const double2 h0 = __ldg(p + 3), h1 = __ldg(p + 4), h2 = __ldg(p + 5);
    const double f = __ddiv_rn(__dsub_rn(h0.x, q), __dsub_rn(h0.x, l0.x));
    A.a0 = __fma_rn(__fma_rn(-f, __dsub_rn(h0.y, l0.y), h0.y), conc, A.a0);
    A.a1 = __fma_rn(__fma_rn(-f, __dsub_rn(h1.x, l1.x), h1.x), conc, A.a1);
    A.a2 = __fma_rn(__fma_rn(-f, __dsub_rn(h1.y, l1.y), h1.y), conc, A.a2);
    A.a3 = __fma_rn(__fma_rn(-f, __dsub_rn(h2.x, l2.x), h2.x), conc, A.a3);
    A.a4 = __fma_rn(__fma_rn(-f, __dsub_rn(h2.y, l2.y), h2.y), conc, A.a4);
}

// two pairs at once: all 12 loads issued before any arithmetic, the two divisions and
// interpolations independent; accumulation in order a then b (reading R8)
__device__ __forceinline__ void accumulate_pair2(const double *__restrict__ pa, int La, double ca,
                                                 const double *__restrict__ pb, int Lb, double cb, double q, Acc &A)
{
    const double2 *p = reinterpret_cast<const double2 *>(pa) + (uint32_t)La * 3;
    const double2 *s = reinterpret_cast<const double2 *>(pb) + (uint32_t)Lb * 3;
    const double2 l0 = __ldg(p + 0), l1 = __ldg(p + 1), l2 = __ldg(p + 2);
    const double2 h0 = __ldg(p + 3), h1 = __ldg(p + 4), h2 = __ldg(p + 5);
    const double2 m0 = __ldg(s + 0), m1 = __ldg(s + 1), m2 = __ldg(s + 2);
    const double2 k0 = __ldg(s + 3), k1 = __ldg(s + 4), k2 = __ldg(s + 5);
    const double fa = __ddiv_rn(__dsub_rn(h0.x, q), __dsub_rn(h0.x, l0.x));
    const double fb = __ddiv_rn(__dsub_rn(k0.x, q), __dsub_rn(k0.x, m0.x));
    const double a0 = __fma_rn(-fa, __dsub_rn(h0.y, l0.y), h0.y), b0 = __fma_rn(-fb, __dsub_rn(k0.y, m0.y), k0.y);
    const double a1 = __fma_rn(-fa, __dsub_rn(h1.x, l1.x), h1.x), b1 = __fma_rn(-fb, __dsub_rn(k1.x, m1.x), k1.x);
    const double a2 = __fma_rn(-fa, __dsub_rn(h1.y, l1.y), h1.y), b2 = __fma_rn(-fb, __dsub_rn(k1.y, m1.y), k1.y);
    const double a3 = __fma_rn(-fa, __dsub_rn(h2.x, l2.x), h2.x), b3 = __fma_rn(-fb, __dsub_rn(k2.x, m2.x), k2.x);
    const double a4 = __fma_rn(-fa, __dsub_rn(h2.y, l2.y), h2.y), b4 = __fma_rn(-fb, __dsub_rn(k2.y, m2.y), k2.y);
    A.a0 = __fma_rn(b0, cb, __fma_rn(a0, ca, A.a0));
    A.a1 = __fma_rn(b1, cb, __fma_rn(a1, ca, A.a1));
    A.a2 = __fma_rn(b2, cb, __fma_rn(a2, ca, A.a2));
    A.a3 = __fma_rn(b3, cb, __fma_rn(a3, ca, A.a3));
    A.a4 = __fma_rn(b4, cb, __fma_rn(a4, ca, A.a4));
}

#endif

// verification value (R10): 1 + first maximum, strict '>' from -1.0
__device__ __forceinline__ uint32_t verify(const Acc &A)
{
    double mx = -1.0;
    uint32_t v = 0;
    if (A.a0 > mx) { mx = A.a0; v = 0; }
    if (A.a1 > mx) { mx = A.a1; v = 1; }
    if (A.a2 > mx) { mx = A.a2; v = 2; }
    if (A.a3 > mx) { mx = A.a3; v = 3; }
    if (A.a4 > mx) { mx = A.a4; v = 4; }
    return v + 1;
}

__device__ __forceinline__ void store_macro(double *__restrict__ out, uint32_t r, const Acc &A)
{
    double *o = out + (size_t)r * 5;
    o[0] = A.a0;
    o[1] = A.a1;
    o[2] = A.a2;
    o[3] = A.a3;
    o[4] = A.a4;
}

// fused epilogue: CTA reduction of (hash, pairs), one 64-bit atomic per counter per CTA
template <int TPB>
__device__ __forceinline__ void reduce_stats(uint32_t my_hash, uint32_t my_pairs, unsigned long long *stats)
{
    __shared__ uint32_t s_red[2][TPB / 32];
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

} // namespace xs
