// lookup_staged.cu -- XS_SEARCH_S: the sorted lookup kernel with staged warp windows
// (DESIGN.md §6.5c).  A persistent grid (2 CTAs of 256 threads per SM); each warp pulls work
// chunks of kStChunk = 256 consecutive sorted slots from an atomic counter and takes
// 32 x kLpl = 128 of them (4 per lane) per iteration; for each material among them (in
// sorted order almost always one) the lanes of that material form the window [q_lo, q_hi]
// and every nuclide of the material is resolved through a window of interval records staged
// in shared memory.
#include <algorithm>
#include <cstddef>

#include "lookup_common.cuh"

namespace xs {

#ifndef XS_S_TPB
#define XS_S_TPB 256
#endif
constexpr int kStTpb = XS_S_TPB;
#ifndef XS_S_MIN_BLOCKS
#define XS_S_MIN_BLOCKS 2
#endif
#ifndef XS_S_CHUNK
#define XS_S_CHUNK 256
#endif
constexpr int kStChunk = XS_S_CHUNK; // sorted slots per work chunk (a warp pulls one at a time)
#ifndef XS_S_LPL
#define XS_S_LPL 4
#endif
#ifndef XS_S_PF
#define XS_S_PF 1
#endif
#ifndef XS_S_WSORT
#define XS_S_WSORT 0
#endif
#ifndef XS_S_STAGE2
#define XS_S_STAGE2 1
#endif
#ifndef XS_S_CNT2
#define XS_S_CNT2 1
#endif
#ifndef XS_S_FASTMASK
#define XS_S_FASTMASK 1
#endif
#ifndef XS_S_ALL
#define XS_S_ALL 1
#endif
#ifndef XS_S_OMETA
#define XS_S_OMETA 1
#endif
#ifndef XS_S_FASTPAIR
#define XS_S_FASTPAIR 1 // one-interval nuclides in pairs (large-U lookup 7.72 -> 7.47 ms; quads 7.53)
#endif
#ifndef XS_S_FASTGRIDS
#define XS_S_FASTGRIDS 1 // grids (bit XS_UNIONIZED = 0, XS_NUCLIDE = 1, XS_HASH = 2) with the one-interval loop
#endif
#ifndef XS_S_FASTPF
#define XS_S_FASTPF 1 // the fast loop's descriptors from lane registers (large-U 7.82 -> 7.73 ms)
#endif
constexpr int kLpl = XS_S_LPL; // lookups per lane per iteration: they share the staged windows

// ---- XS_SEARCH_S: staged warp windows -----------------------------------
// Per warp in dynamic shared memory: kStageCap interval records, their upper energies again
// in a compact array (the window count reads them), 32 window descriptors and the owner
// lane of every staged interval.  Interval record (112 B = 7 x 16 B): the quantities of
// reading R8 that do not depend on q, rounded exactly as accumulate_pair rounds them,
//   [0] E_hi  [1] conc of the nuclide  [2] d = E_hi - E_lo  [3] y = RN(1/d)
//   [4 + 2c] X_c,hi  [5 + 2c] dX_c = X_c,hi - X_c,lo
// so a pair costs one subtraction, Markstein's quotient (3 ops) and 10 FMAs.
#ifndef XS_STAGE_CAP
#define XS_STAGE_CAP 48
#endif
constexpr int kStageCap = XS_STAGE_CAP; // intervals per warp
static_assert(!XS_S_STAGE2 || kStageCap <= 64, "the two-interval staging covers at most 64 intervals per pass");
#ifndef XS_S_SORT_MIN
#define XS_S_SORT_MIN 64
#endif
constexpr int kSortMinNucs = XS_S_SORT_MIN; // sort a warp's lookups when their material has >= this many nuclides
constexpr int kIvDoubles = 14;
// XS_S_TMA applies to the hash grid (XL): bulk-copied records took XL's lookup kernel from
// 19.33 to 18.42 ms but the nuclide / unionized ones 2-6% slower (their windows are mostly
// one interval, staging is cheap there, and the 112 B records double the L2 footprint of 48 B
// points) -- DESIGN.md §6.8
template <int GRID> constexpr bool kTma = kTmaStage && GRID == XS_HASH;
template <int GRID> constexpr int kEhStride = kTma<GRID> ? kIvDoubles : 1; // stride of the upper energies
// stage_interval reads points k and k+1 of a 48 B point-record row; the XS_IV build points
// NucRef.pts at 96 B interval records instead, which this kernel does not stage
static_assert(!kIv, "XS_SEARCH_S stages 48 B point records: build without -DXS_IV");
static_assert(kIvDoubles * 8 % 16 == 0, "bulk copies move whole 16 B units");

struct alignas(16) StageMeta {
    double conc;
    int32_t lo;     // L(q_min) of the nuclide
    int32_t offcnt; // (first staged interval << 16) | intervals, or -1: not staged
};
static_assert(sizeof(StageMeta) == 16 && offsetof(StageMeta, offcnt) == 12, "the hot loop reads offcnt at byte 12");
constexpr int kStageWarpBytes = kStageCap * kIvDoubles * 8 + kStageCap * 8 + 32 * (int)sizeof(StageMeta) +
                                32 * 8 + 32 * 4 + ((kStageCap + 15) / 16) * 16 + 16;

// The group's per-nuclide state lives in shared memory, not in registers, while the
// group is computed (registers decide the occupancy of this kernel).
struct WarpStage {
    double *rec;         // [kStageCap][kIvDoubles]
    double *eh;          // [kStageCap] E_hi of each staged interval
    StageMeta *meta;     // [32] conc, lo, staged position
    const double **pts;  // [32] point row of the nuclide
    int *cnt;            // [32] intervals of the nuclide's window
    uint8_t *owner;      // [kStageCap]
    uint64_t *mbar;      // XS_S_TMA: the warp's mbarrier for the bulk copies of a pass
    // the hot loop's view: byte offsets into st_smem (32-bit shared addressing; generic 64-bit
    // pointers were rematerialised from SR_TID / SR_CgaCtaId for every nuclide)
    int orec, oeh, ometa;
};

extern __shared__ __align__(16) unsigned char st_smem[]; // k_lookup_staged's dynamic shared memory

__device__ __forceinline__ WarpStage warp_stage(unsigned char *smem)
{
    WarpStage w;
    unsigned char *base = smem + (threadIdx.x >> 5) * kStageWarpBytes;
    w.rec = reinterpret_cast<double *>(base);
    w.eh = w.rec + kStageCap * kIvDoubles;
    w.meta = reinterpret_cast<StageMeta *>(w.eh + kStageCap);
    w.pts = reinterpret_cast<const double **>(w.meta + 32);
    w.cnt = reinterpret_cast<int *>(w.pts + 32);
    w.owner = reinterpret_cast<uint8_t *>(w.cnt + 32);
    w.mbar = reinterpret_cast<uint64_t *>(w.owner + ((kStageCap + 15) / 16) * 16);
    // opaque: kept in registers, not re-derived from SR_TID.X (a long-latency S2R) per nuclide
    int o = (int)(threadIdx.x >> 5) * kStageWarpBytes;
    asm("mov.b32 %0, %0;" : "+r"(o));
    w.orec = o;
    w.oeh = o + kStageCap * kIvDoubles * 8;
    w.ometa = w.oeh + kStageCap * 8;
    return w;
}

// ---- XS_S_TMA: interval records copied by the bulk-copy engine (cp.async.bulk, UBLKCP) ----
__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *mb)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(mb)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *mb, unsigned bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(mb)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *mb, unsigned phase)
{
    asm volatile("{\n\t.reg .pred P;\n"
                 "XS_WAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
                 "@!P bra XS_WAIT_%=;\n\t}" ::"r"(smem_u32(mb)), "r"(phase) : "memory");
}

// `bytes` (a multiple of 16) from global `src` to shared `dst` (both 16 B aligned), completing
// on the mbarrier's transaction count
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *mb)
{
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(mb)) : "memory");
}

// f = RN(a / d) from y = RN(1/d): q0 = RN(a y), r = a - d q0 (exact, an FMA), f = RN(q0 + r y).
// Markstein's theorem: with y within half an ulp of 1/d and q0 within one ulp of a/d (both
// hold here, and a, d are far from under/overflow: multiples of 2^-63 in (-1, 1)), f is the
// correctly rounded quotient, i.e. bit-identical to IEEE division (__ddiv_rn); pinned on the
// CPU by tests/test_markstein.py, and by every bit-exact parity test of XS_SEARCH_S.
__device__ __forceinline__ double quotient_markstein(double a, double d, double y)
{
    const double q0 = __dmul_rn(a, y);
    const double r = __fma_rn(-d, q0, a);
    return __fma_rn(r, y, q0);
}

// a staged interval record in registers
struct IvRec {
    double2 e, dy, x0, x1, x2, x3, x4;
};

__device__ __forceinline__ IvRec load_rec(const double *R)
{
    const double2 *p = reinterpret_cast<const double2 *>(R);
    return IvRec{p[0], p[1], p[2], p[3], p[4], p[5], p[6]};
}

// the interpolation of accumulate_pair (reading R8; identical results) from a staged
// interval record
__device__ __forceinline__ void accumulate_interval(const IvRec &v, double q, double conc, Acc &A)
{
    const double f = quotient_markstein(__dsub_rn(v.e.x, q), v.dy.x, v.dy.y);
    A.a0 = __fma_rn(__fma_rn(-f, v.x0.y, v.x0.x), conc, A.a0);
    A.a1 = __fma_rn(__fma_rn(-f, v.x1.y, v.x1.x), conc, A.a1);
    A.a2 = __fma_rn(__fma_rn(-f, v.x2.y, v.x2.x), conc, A.a2);
    A.a3 = __fma_rn(__fma_rn(-f, v.x3.y, v.x3.x), conc, A.a3);
    A.a4 = __fma_rn(__fma_rn(-f, v.x4.y, v.x4.x), conc, A.a4);
}

// interval record k of a point row (points k and k+1) into shared memory
struct RawIv { // points k and k+1 of a 48 B point-record row
    double2 a0, a1, a2, b0, b1, b2;
};

__device__ __forceinline__ RawIv load_raw(const double *__restrict__ pts, int k)
{
    const double2 *p = reinterpret_cast<const double2 *>(pts) + (size_t)(uint32_t)k * 3;
    return RawIv{__ldg(p), __ldg(p + 1), __ldg(p + 2), __ldg(p + 3), __ldg(p + 4), __ldg(p + 5)};
}

__device__ __forceinline__ void store_interval(const RawIv &v, double *dst, double *eh, double conc)
{
    const double2 a0 = v.a0, a1 = v.a1, a2 = v.a2, b0 = v.b0, b1 = v.b1, b2 = v.b2;
    const double d = __dsub_rn(b0.x, a0.x);
    double2 *o = reinterpret_cast<double2 *>(dst) + 1;
    o[-1] = make_double2(b0.x, conc); // the nuclide's concentration rides in the pad slot
    o[0] = make_double2(d, __drcp_rn(d));
    o[1] = make_double2(b0.y, __dsub_rn(b0.y, a0.y));
    o[2] = make_double2(b1.x, __dsub_rn(b1.x, a1.x));
    o[3] = make_double2(b1.y, __dsub_rn(b1.y, a1.y));
    o[4] = make_double2(b2.x, __dsub_rn(b2.x, a2.x));
    o[5] = make_double2(b2.y, __dsub_rn(b2.y, a2.y));
    *eh = b0.x;
}

__device__ __forceinline__ void stage_interval(const double *__restrict__ pts, int k, double *dst, double *eh,
                                               double conc)
{
    store_interval(load_raw(pts, k), dst, eh, conc);
}

// c = #{k in 1..cnt-1 : E[lo + k] <= q} (E[lo + k] = eh[k - 1]), i.e. L(q) - lo: short
// windows by three compares of values shared by the lane's lookups, longer ones by Listing 1
// (U1) over eh
template <int EHS>
__device__ __forceinline__ int window_count(const double *eh, int cnt, double q)
{
    int c = 0, len = cnt;
    while (len > 1) {
        const int h = len >> 1;
        if (eh[(c + h - 1) * EHS] > q) {
            len = h;
        } else {
            c += h;
            len -= h;
        }
    }
    return c;
}

// Bitonic sort of the warp's kLpl x 32 (key, value) pairs (kLpl a power of two), ascending
// over the position e = l * 32 + lane (element l of a lane).  Equal keys keep their own
// values on both sides of an exchange, so the result is a permutation.
__device__ __forceinline__ void warp_sort(uint64_t (&k)[kLpl], uint32_t (&v)[kLpl])
{
    static_assert((kLpl & (kLpl - 1)) == 0, "warp_sort needs a power-of-two kLpl");
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int size = 2; size <= 32 * kLpl; size <<= 1) {
#pragma unroll
        for (int j = size >> 1; j > 0; j >>= 1) {
            if (j >= 32) { // the partner is element l ^ (j / 32) of this lane
                const int jl = j >> 5;
#pragma unroll
                for (int l = 0; l < kLpl; l++) {
                    if ((l & jl) == 0) {
                        const int l2 = l | jl;
                        const bool asc = ((l * 32) & size) == 0;
                        if (asc ? k[l2] < k[l] : k[l2] > k[l]) {
                            const uint64_t tk = k[l];
                            k[l] = k[l2];
                            k[l2] = tk;
                            const uint32_t tv = v[l];
                            v[l] = v[l2];
                            v[l2] = tv;
                        }
                    }
                }
            } else {
#pragma unroll
                for (int l = 0; l < kLpl; l++) {
                    const int e = l * 32 + lane;
                    const uint64_t ko = __shfl_xor_sync(0xffffffffu, k[l], j);
                    const uint32_t vo = __shfl_xor_sync(0xffffffffu, v[l], j);
                    const bool keep_min = ((e & j) == 0) == ((e & size) == 0);
                    if (keep_min ? ko < k[l] : ko > k[l]) {
                        k[l] = ko;
                        v[l] = vo;
                    }
                }
            }
        }
    }
}

// One nuclide of a staged group for the lookups in `mine` (ascending nuclide order, R8):
// the window's interval records are at rec_all + (m.offcnt >> 16) (its upper energies at
// eh_all + ...); a nuclide whose window was not staged (m.offcnt < 0) takes the per-lane H
// path.  `col` is the nuclide's column in out_idx.
template <int GRID, bool OUTS, bool ALL = false>
__device__ __forceinline__ void compute_nuclide(const GridView &gv, int ref_idx, int col, const int offcnt,
                                                const StageMeta *mp, int oeh, int orec,
                                                const bool (&mine)[kLpl], const double (&q)[kLpl],
                                                const uint32_t (&r)[kLpl], int32_t *__restrict__ out_idx,
                                                Acc (&A)[kLpl])
{
    if (offcnt >= 0) {
        const int off_w = offcnt >> 16, cnt_w = offcnt & 0xFFFF;
        const double *R = reinterpret_cast<const double *>(st_smem + orec) + off_w * kIvDoubles;
        // upper energies E[lo + k] = eh[(k - 1) kEhStride]: the compact array, or (bulk-copied
        // records) the records' own first field
        const double *eh = kTma<GRID> ? R : reinterpret_cast<const double *>(st_smem + oeh) + off_w;
        // the nuclide's concentration: in the record's pad slot, or (bulk-copied records, which
        // are shared by every material) from the descriptor
        const double conc = kTma<GRID> ? mp->conc : 0.0;
        // branch-free over the lane's lookups, so their FP64 chains interleave: a lookup
        // that is not `mine` accumulates with concentration +0, fma(micro, +0, acc) == acc
        // exactly (micro is finite and acc is never -0)
        if (cnt_w == 1) { // one interval: its record is loaded once for the lane's lookups
            const IvRec v = load_rec(R);
#pragma unroll
            for (int l = 0; l < kLpl; l++) {
                accumulate_interval(v, q[l], (ALL || mine[l]) ? (kTma<GRID> ? conc : v.e.y) : 0.0, A[l]);
                if constexpr (OUTS) {
                    if (out_idx && mine[l])
                        out_idx[(size_t)r[l] * gv.max_nucs + col] = mp->lo;
                }
            }
        } else if (cnt_w <= 4) { // the upper energies of a short window, shared by the lookups
            const double inf = __longlong_as_double(0x7FF0000000000000ll);
            const double e1 = eh[0];
            const double e2 = cnt_w > 2 ? eh[kEhStride<GRID>] : inf;
            const double e3 = cnt_w > 3 ? eh[2 * kEhStride<GRID>] : inf;
#pragma unroll
            for (int l = 0; l < kLpl; l++) {
                // E[lo + k] = eh[k - 1], k = 1..cnt-1 ascending: c = #{e_k <= q} by two
                // compares (e2 first, then e3 or e1) instead of three
#if XS_S_CNT2
                const bool p2 = e2 <= q[l];
                const double e = p2 ? e3 : e1;
                const int c = (p2 ? 2 : 0) + (e <= q[l] ? 1 : 0);
#else
                const int c = (e1 <= q[l] ? 1 : 0) + (e2 <= q[l] ? 1 : 0) + (e3 <= q[l] ? 1 : 0);
#endif
                const IvRec v = load_rec(R + c * kIvDoubles);
                accumulate_interval(v, q[l], (ALL || mine[l]) ? (kTma<GRID> ? conc : v.e.y) : 0.0, A[l]);
                if constexpr (OUTS) {
                    if (out_idx && mine[l])
                        out_idx[(size_t)r[l] * gv.max_nucs + col] = mp->lo + c;
                }
            }
        } else {
#pragma unroll
            for (int l = 0; l < kLpl; l++) {
                if (mine[l]) {
                    const int c = window_count<kEhStride<GRID>>(eh, cnt_w, q[l]);
                    const IvRec v = load_rec(R + c * kIvDoubles);
                    accumulate_interval(v, q[l], kTma<GRID> ? conc : v.e.y, A[l]);
                    if constexpr (OUTS) {
                        if (out_idx)
                            out_idx[(size_t)r[l] * gv.max_nucs + col] = mp->lo + c;
                    }
                }
            }
        }
    } else {
        const Row rw = load_row(gv, ref_idx);
#pragma unroll
        for (int l = 0; l < kLpl; l++) {
            if (mine[l]) {
                int e_me = 0;
                if constexpr (GRID == XS_UNIONIZED)
                    e_me = union_index<GRID, XS_SEARCH_S>(gv, q[l]);
                const int L = lower_index<GRID, XS_SEARCH_S>(gv, rw, q[l], e_me);
                accumulate_pair(rw.pts, L, q[l], rw.conc, A[l]);
                if constexpr (OUTS) {
                    if (out_idx)
                        out_idx[(size_t)r[l] * gv.max_nucs + col] = L;
                }
            }
        }
    }
}

// The lookups in `mine` (one material: row `roww`, nn nuclides; kLpl per lane) accumulate
// every nuclide of the material.  All 32 lanes call it (warp collectives inside).
template <int GRID, bool OUTS>
__device__ __forceinline__ void staged_material(const GridView &gv, unsigned &tma_phase, int roww, int nn, const bool (&mine)[kLpl],
                                                const double (&q)[kLpl], const uint32_t (&r)[kLpl],
                                                const WarpStage &ws, int32_t *__restrict__ out_idx,
                                                Acc (&A)[kLpl])
{
    const int lane = threadIdx.x & 31;
    // every lookup of the material has q in [q_lo, q_hi] and L is monotone, so
    // L(q) = L(q_lo) + #{k in (L(q_lo), L(q_hi)] : E[k] <= q}
    double mn = __longlong_as_double(0x7FF0000000000000ll), mx = -1.0;
#pragma unroll
    for (int l = 0; l < kLpl; l++) {
        mn = mine[l] ? fmin(mn, q[l]) : mn;
        mx = mine[l] ? fmax(mx, q[l]) : mx;
    }
    const double q_lo = warp_min(mn), q_hi = warp_max(mx);
#if XS_S_ALL
    bool mine_all = true;
#pragma unroll
    for (int l = 0; l < kLpl; l++)
        mine_all = mine_all && mine[l];
    const bool all_mine = __all_sync(0xffffffffu, mine_all);
#endif
    int e_lo = 0, e_hi = 0;
    if constexpr (GRID == XS_UNIONIZED) {
        e_lo = union_index<GRID, XS_SEARCH_S>(gv, q_lo);
        e_hi = union_index<GRID, XS_SEARCH_S>(gv, q_hi);
    }
    for (int g0 = 0; g0 < nn; g0 += 32) {
        // lane t: the window of nuclide g0 + t (H bounds), intervals lo .. lo + cnt - 1
        const int ng = min(32, nn - g0);
        __syncwarp(); // the previous group's shared-memory reads are done
        if (lane < ng) {
            const Row rw = load_row(gv, roww + g0 + lane);
            const int lo = lower_index<GRID, XS_SEARCH_S>(gv, rw, q_lo, e_lo);
            ws.cnt[lane] = lower_index<GRID, XS_SEARCH_S>(gv, rw, q_hi, e_hi) - lo + 1;
            ws.meta[lane] = StageMeta{rw.conc, lo, 0};
            ws.pts[lane] = kTma<GRID> ? gv.ivs + (size_t)rw.nuc * (uint32_t)(gv.n - 1) * kIvDoubles : rw.pts;
        }
        __syncwarp();
        for (int b0 = 0; b0 < ng;) { // passes over the group (warp-uniform)
            const int want = (lane >= b0 && lane < ng) ? ws.cnt[lane] : 0;
            int incl = want;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(0xffffffffu, incl, o);
                incl += (lane >= o) ? t : 0;
            }
            const bool fits = want > 0 && incl <= kStageCap; // lanes b0 .. b1-1
            const int nfit = __popc(__ballot_sync(0xffffffffu, fits));
            const int T = nfit ? __shfl_sync(0xffffffffu, incl, b0 + nfit - 1) : 0; // intervals staged
            int b1 = b0 + nfit;
            __syncwarp(); // the previous pass's shared-memory reads are done
            if (fits) {
                const int off = incl - want;
                ws.meta[lane].offcnt = (off << 16) | want;
                for (int k = 0; k < want; k++)
                    ws.owner[off + k] = (uint8_t)lane;
            }
            if (b1 == b0) { // nuclide b0's window alone exceeds the stage: per-lane H path
                if (lane == b0)
                    ws.meta[lane].offcnt = -1;
                b1 = b0 + 1;
            }
            __syncwarp();
            // interval i of the pass is staged by lane i % 32: owner nuclide j, its k-th interval
            if constexpr (kTma<GRID>) {
                // the pass's windows are contiguous runs of precomputed records (gv.ivs): each
                // nuclide's lane issues one bulk copy of its window, the warp waits on its
                // mbarrier for all of them (T intervals x 112 B); no registers, no LSU traffic
                if (T > 0) {
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); // prior reads before async writes
                    if (lane == 0)
                        mbar_expect_tx(ws.mbar, (unsigned)T * kIvDoubles * 8);
                    __syncwarp();
                    if (fits) {
                        const int off = incl - want;
                        bulk_g2s(ws.rec + off * kIvDoubles, ws.pts[lane] + (size_t)(uint32_t)ws.meta[lane].lo * kIvDoubles,
                                 (unsigned)want * kIvDoubles * 8, ws.mbar);
                    }
                    mbar_wait(ws.mbar, tma_phase);
                    tma_phase ^= 1u;
                }
            } else {
#if XS_S_STAGE2
            // each lane stages intervals lane and lane + 32 (T <= kStageCap <= 64): the second
            // interval's six loads are issued with the first's, so a pass waits for one
            // memory latency instead of two
            {
                const int i1 = lane + 32;
                const bool h0 = lane < T, h1 = i1 < T;
                const int j0 = h0 ? ws.owner[lane] : 0, j1 = h1 ? ws.owner[i1] : 0;
                const StageMeta m0 = ws.meta[j0], m1 = ws.meta[j1];
                RawIv v0{}, v1{};
                if (h0)
                    v0 = load_raw(ws.pts[j0], m0.lo + (lane - (m0.offcnt >> 16)));
                if (h1)
                    v1 = load_raw(ws.pts[j1], m1.lo + (i1 - (m1.offcnt >> 16)));
                if (h0)
                    store_interval(v0, ws.rec + lane * kIvDoubles, ws.eh + lane, m0.conc);
                if (h1)
                    store_interval(v1, ws.rec + i1 * kIvDoubles, ws.eh + i1, m1.conc);
            }
#else
            for (int i = lane; i < T; i += 32) {
                const int j = ws.owner[i];
                const StageMeta mj = ws.meta[j];
                stage_interval(ws.pts[j], mj.lo + (i - (mj.offcnt >> 16)), ws.rec + i * kIvDoubles, ws.eh + i, mj.conc);
            }
#endif
            }
            __syncwarp();
            // the descriptors through the warp's opaque 32-bit offset (a generic pointer into the
            // stage was rematerialised from SR_TID / SR_CgaCtaId at every use; the bulk-copied
            // records of the hash grid read their concentration from it: XL 18.37 -> 18.00 ms)
            const StageMeta *OMETA = (XS_S_OMETA && kTma<GRID>) ? reinterpret_cast<const StageMeta *>(st_smem + ws.ometa)
                                                                : ws.meta;
            // ascending nuclide order (R8); the next nuclide's window descriptor is read one
            // nuclide ahead (the record load depends on it)
            // the offcnt words of the pass's nuclides: StageMeta is 16 B, offcnt at byte 12
            const int *ocp = reinterpret_cast<const int *>(st_smem + ws.ometa + 12);
            int oc = ocp[4 * b0];
#if XS_S_ALL
            if (all_mine) { // every lookup of the warp is this material's (the sorted norm): no selects
#if XS_S_FASTMASK
                // the pass's one-interval windows as a warp-uniform bit mask (a ballot): the
                // common step -- one record for the lane's lookups -- branches on a uniform bit
                // instead of re-deciding a possibly divergent branch per nuclide
                // (worth it where one-interval windows dominate -- the unionized configuration's
                // 100M lookups: large-U 8.04 -> 7.91 ms; compiled into the nuclide / hash kernels
                // it cost small / large / XL 0.5-2% through their register allocation)
                if constexpr (((XS_S_FASTGRIDS >> GRID) & 1) && !OUTS) {
                    const int myoc = (lane >= b0 && lane < b1) ? ocp[4 * lane] : -1;
                    const unsigned fast = __ballot_sync(0xffffffffu, myoc >= 0 && (myoc & 0xFFFF) == 1);
#if XS_S_FASTPAIR
                    // two consecutive one-interval nuclides per iteration (their records are
                    // adjacent in the stage): one loop test and one shuffle per pair
                    for (int jj = b0; jj < b1;) {
                        const int ocj = __shfl_sync(0xffffffffu, myoc, jj);
#if XS_S_FASTPAIR >= 4
                        if (((fast >> jj) & 15u) == 15u && jj + 3 < b1) {
                            const double *R = reinterpret_cast<const double *>(st_smem + ws.orec) +
                                              (ocj >> 16) * kIvDoubles;
#pragma unroll
                            for (int u = 0; u < 4; u++) {
                                const IvRec v = load_rec(R + u * kIvDoubles);
#pragma unroll
                                for (int l = 0; l < kLpl; l++)
                                    accumulate_interval(v, q[l], v.e.y, A[l]);
                            }
                            jj += 4;
                        } else
#endif
                        if (((fast >> jj) & 3u) == 3u && jj + 1 < b1) {
                            const double *R = reinterpret_cast<const double *>(st_smem + ws.orec) +
                                              (ocj >> 16) * kIvDoubles;
                            {
                                const IvRec v = load_rec(R);
#pragma unroll
                                for (int l = 0; l < kLpl; l++)
                                    accumulate_interval(v, q[l], v.e.y, A[l]);
                            }
                            {
                                const IvRec v = load_rec(R + kIvDoubles);
#pragma unroll
                                for (int l = 0; l < kLpl; l++)
                                    accumulate_interval(v, q[l], v.e.y, A[l]);
                            }
                            jj += 2;
                        } else if ((fast >> jj) & 1u) {
                            const double *R = reinterpret_cast<const double *>(st_smem + ws.orec) +
                                              (ocj >> 16) * kIvDoubles;
                            const IvRec v = load_rec(R);
#pragma unroll
                            for (int l = 0; l < kLpl; l++)
                                accumulate_interval(v, q[l], v.e.y, A[l]);
                            jj++;
                        } else {
                            compute_nuclide<GRID, OUTS, true>(gv, roww + g0 + jj, g0 + jj, ocj, OMETA + jj,
                                                              ws.oeh, ws.orec, mine, q, r, out_idx, A);
                            jj++;
                        }
                    }
#elif XS_S_FASTPF
                    // the descriptors of the pass are already in lane registers (myoc): the
                    // record address comes from a shuffle, not a dependent shared-memory load
                    for (int jj = b0; jj < b1; jj++) {
                        const int ocj = __shfl_sync(0xffffffffu, myoc, jj);
                        if ((fast >> jj) & 1u) {
                            const double *R = reinterpret_cast<const double *>(st_smem + ws.orec) +
                                              (ocj >> 16) * kIvDoubles;
                            const IvRec v = load_rec(R);
                            const double conc = kTma<GRID> ? OMETA[jj].conc : v.e.y;
#pragma unroll
                            for (int l = 0; l < kLpl; l++)
                                accumulate_interval(v, q[l], conc, A[l]);
                        } else {
                            compute_nuclide<GRID, OUTS, true>(gv, roww + g0 + jj, g0 + jj, ocj, OMETA + jj,
                                                              ws.oeh, ws.orec, mine, q, r, out_idx, A);
                        }
                    }
#else
                    for (int jj = b0; jj < b1; jj++) {
                        if ((fast >> jj) & 1u) {
                            const double *R = reinterpret_cast<const double *>(st_smem + ws.orec) +
                                              (ocp[4 * jj] >> 16) * kIvDoubles;
                            const IvRec v = load_rec(R);
                            const double conc = kTma<GRID> ? OMETA[jj].conc : v.e.y;
#pragma unroll
                            for (int l = 0; l < kLpl; l++)
                                accumulate_interval(v, q[l], conc, A[l]);
                        } else {
                            compute_nuclide<GRID, OUTS, true>(gv, roww + g0 + jj, g0 + jj, ocp[4 * jj], OMETA + jj,
                                                              ws.oeh, ws.orec, mine, q, r, out_idx, A);
                        }
                    }
#endif
                } else
#endif
                for (int jj = b0; jj < b1; jj++) {
                    const int oc_next = jj + 1 < b1 ? ocp[4 * (jj + 1)] : 0;
                    compute_nuclide<GRID, OUTS, true>(gv, roww + g0 + jj, g0 + jj, oc, OMETA + jj, ws.oeh, ws.orec,
                                                      mine, q, r, out_idx, A);
                    oc = oc_next;
                }
            } else
#endif
                for (int jj = b0; jj < b1; jj++) {
                    const int oc_next = jj + 1 < b1 ? ocp[4 * (jj + 1)] : 0;
                    compute_nuclide<GRID, OUTS>(gv, roww + g0 + jj, g0 + jj, oc, OMETA + jj, ws.oeh, ws.orec, mine,
                                                q, r, out_idx, A);
                    oc = oc_next;
                }
            b0 = b1;
        }
    }
}

// The S path for one warp's kLpl x 32 lookups (act: lane has a lookup; mat per lookup): an
// optional warp energy sort, then one staged_material round per material among them.
template <int GRID, bool OUTS>
__device__ __forceinline__ void warp_lookups(const GridView &gv, unsigned &tma_phase, const WarpStage &ws, bool (&act)[kLpl],
                                             double (&q)[kLpl], uint32_t (&r)[kLpl], int (&mat)[kLpl],
                                             int32_t *__restrict__ out_idx, Acc (&A)[kLpl])
{
    const int lane = threadIdx.x & 31;
    bool mine[kLpl];
    unsigned todo[kLpl];
#if XS_S_WSORT
    {
        // one material (the sorted norm): order the warp's lookups by energy, so each
        // element l covers a slice of the energy band and an interval-record load touches
        // fewer distinct records (shared-memory wavefronts bound S)
        const int mat0 = __shfl_sync(0xffffffffu, mat[0], 0);
        bool same = true;
#pragma unroll
        for (int l = 0; l < kLpl; l++)
            same = same && (!act[l] || mat[l] == mat0);
        if (__ldg(gv.num_nucs + mat0) >= kSortMinNucs && __all_sync(0xffffffffu, same)) {
            int n_act = 0;
#pragma unroll
            for (int l = 0; l < kLpl; l++)
                n_act += __popc(__ballot_sync(0xffffffffu, act[l]));
            uint64_t key[kLpl];
            uint32_t val[kLpl];
#pragma unroll
            for (int l = 0; l < kLpl; l++) { // q >= 0: its bits order like its value
                key[l] = act[l] ? (uint64_t)__double_as_longlong(q[l]) : ~0ull;
                val[l] = r[l];
            }
            warp_sort(key, val);
#pragma unroll
            for (int l = 0; l < kLpl; l++) {
                act[l] = l * 32 + lane < n_act;
                q[l] = act[l] ? __longlong_as_double((long long)key[l]) : 0.0;
                r[l] = val[l];
                mat[l] = act[l] ? mat0 : 0;
            }
        }
    }
#endif
#pragma unroll
    for (int l = 0; l < kLpl; l++)
        todo[l] = __ballot_sync(0xffffffffu, act[l]);
    // one round per material among the warp's lookups (sorted: almost always one)
    for (;;) {
        int src = -1;
#pragma unroll
        for (int l = kLpl - 1; l >= 0; l--)
            src = todo[l] ? l * 32 + __ffs(todo[l]) - 1 : src;
        if (src < 0)
            break;
        int mw = mat[0];
#pragma unroll
        for (int l = 1; l < kLpl; l++)
            mw = (src >> 5) == l ? mat[l] : mw;
        const int mat_w = __shfl_sync(0xffffffffu, mw, src & 31);
#pragma unroll
        for (int l = 0; l < kLpl; l++) {
            mine[l] = act[l] && mat[l] == mat_w;
            todo[l] &= ~__ballot_sync(0xffffffffu, mine[l]);
        }
        staged_material<GRID, OUTS>(gv, tma_phase, mat_w * gv.max_nucs, __ldg(gv.num_nucs + mat_w), mine, q, r, ws,
                                    out_idx, A);
    }
}

template <int GRID, bool OUTS>
__global__ void __launch_bounds__(kStTpb, XS_S_MIN_BLOCKS)
    k_lookup_staged(GridView gv, SortedView so, int count_arg, double *__restrict__ out_, int32_t *__restrict__ out_idx_,
                    unsigned long long *__restrict__ stats)
{
    pdl_wait(); // the sort's outputs (and the work counter it zeroed) are complete
    const int count = so.count_dev ? (int)*so.count_dev : count_arg; // a key-range shard's slots
    double *__restrict__ out = OUTS ? out_ : nullptr;
    int32_t *__restrict__ out_idx = OUTS ? out_idx_ : nullptr;
    __shared__ uint32_t s_mb[kMaterials + 1];
    if (threadIdx.x <= kMaterials)
        s_mb[threadIdx.x] = __ldg(so.mb_dev + threadIdx.x);
    __syncthreads();
    const WarpStage ws = warp_stage(st_smem);
    const int lane = threadIdx.x & 31;
    unsigned tma_phase = 0; // XS_S_TMA: parity of the warp's mbarrier phase to wait for
    if (kTma<GRID>) {
        if (lane == 0)
            mbar_init(ws.mbar);
        __syncwarp();
    }
    const uint64_t pol = policy_evict_first();
    uint32_t my_hash = 0, my_pairs = 0;
    for (;;) {
        int c;
        if (lane == 0)
            c = atomicAdd(so.work, 1);
        c = __shfl_sync(0xffffffffu, c, 0);
        if (c * kStChunk >= count)
            break;
#if XS_S_PF
        // chunks are handed out in order: the chunk one resident wave ahead is fetched by some
        // warp about one chunk-time from now -- bring its slots and energies into L2
        if (so.q) {
            const int cp = c + (int)(gridDim.x * (kStTpb / 32));
            constexpr int kQLines = kStChunk * 8 / 128, kSLines = kStChunk * 4 / 128;
            if (lane < kQLines + kSLines && cp * kStChunk < count) {
                const void *a = lane < kQLines ? (const void *)(so.q + (size_t)cp * kStChunk + lane * 16)
                                               : (const void *)(so.slot + (size_t)cp * kStChunk + (lane - kQLines) * 32);
                asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
            }
        }
#endif
        const int jend = min(count, c * kStChunk + kStChunk);
        for (int jw = c * kStChunk; jw < jend; jw += 32 * kLpl) {
            bool act[kLpl];
            double q[kLpl];
            uint32_t r[kLpl];
            int mat[kLpl];
            Acc A[kLpl];
            // material of the iteration's slots: one (warp-uniform) lookup when they all lie
            // in one material's run of slots (the sorted norm), else per lookup
            const int mw = material_of(s_mb, (uint32_t)jw);
            const bool one_mat = (uint32_t)min(jend, jw + 32 * kLpl) <= s_mb[mw + 1];
#pragma unroll
            for (int l = 0; l < kLpl; l++) {
                const int j = jw + l * 32 + lane;
                act[l] = j < jend;
                r[l] = act[l] ? ld_stream(so.slot + j, pol) : 0u;
                q[l] = act[l] ? (so.q ? ld_stream(so.q + j, pol) : ld_stream(so.q_of + r[l], pol)) : 0.0;
                mat[l] = !act[l] ? 0 : (one_mat ? mw : material_of(s_mb, (uint32_t)j));
            }
            warp_lookups<GRID, OUTS>(gv, tma_phase, ws, act, q, r, mat, out_idx, A);
#pragma unroll
            for (int l = 0; l < kLpl; l++) {
                if (act[l]) {
                    my_hash += verify(A[l]);
                    my_pairs += (uint32_t)__ldg(gv.num_nucs + mat[l]);
                    if (out)
                        store_macro(out, r[l], A[l]);
                }
            }
        }
    }
    reduce_stats<kStTpb>(my_hash, my_pairs, stats);
    if (so.pub && threadIdx.x == 0) { // the last CTA publishes the totals to host-mapped memory
        __threadfence();
        if (atomicAdd(so.done, 1u) == gridDim.x - 1) {
            __threadfence();
            const unsigned long long h = atomicAdd(stats + 0, 0ull), pr = atomicAdd(stats + 1, 0ull),
                                     nl = atomicAdd(stats + 2, 0ull);
            volatile unsigned long long *p = so.pub;
            p[0] = h;
            p[1] = pr;
            p[2] = nl;
            __threadfence_system();
        }
    }
}

using StagedFn = void (*)(GridView, SortedView, int, double *, int32_t *, unsigned long long *);

template <int GRID> static StagedFn pick_staged(bool outs)
{
    return outs ? k_lookup_staged<GRID, true> : k_lookup_staged<GRID, false>;
}

void launch_staged(int grid_type, int blocks, int tpb, cudaStream_t stream, const GridView &gv,
                   const SampleView &sv, const SortedView &so, double *out, int32_t *out_idx,
                   unsigned long long *stats)
{
    const bool outs = out || out_idx;
    StagedFn f = grid_type == XS_NUCLIDE     ? pick_staged<XS_NUCLIDE>(outs)
                 : grid_type == XS_UNIONIZED ? pick_staged<XS_UNIONIZED>(outs)
                                             : pick_staged<XS_HASH>(outs);
    (void)tpb; // one configuration: 256 threads, XS_S_MIN_BLOCKS CTAs per SM
    const int smem = (kStTpb / 32) * kStageWarpBytes;
    const int per_sm = resident_ctas((const void *)f, kStTpb, smem);
    const int sms = sm_count_cached();
    const int want = (int)((sv.count + kStTpb - 1) / kStTpb);
    const int nb = std::max(1, std::min(want, sms * std::max(per_sm, 1)));
    (void)blocks;
    launch_pdl(f, nb, kStTpb, smem, stream, gv, so, (int)sv.count, out, out_idx, stats);
    XS_CUDA_TRY(cudaGetLastError());
}

} // namespace xs
