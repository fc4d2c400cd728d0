// sort.cu -- sampling + the (material, energy) counting sort.
//
// Key = kbase[material] + energy bucket (BucketPlan: material m gets nb[m] buckets in
// proportion to P(m) * num_nucs[m], its expected share of the pairs), K <= 49152.
//   k_bucket_count   sample each lookup of the chunk once (one Listing-7 jump per thread,
//                    then one affine step per lookup), write its energy and key at its own
//                    offset (coalesced) and histogram the keys in shared memory
//   k_bucket_colscan per bucket, exclusive scan over CTAs (loads batched by 8)
//   k_bucket_base    exclusive scan of the bucket totals + material bases (one CTA)
//   k_bucket_scatter scatter the 4 B lookup offsets to their slots, one launch per window of
//                    buckets whose slots (16-48 MB) stay L2-resident, so the random
//                    partial-sector writes merge in L2
//   k_bucket_refine  (sorted fused path, the default) per group of buckets: a counting sort of
//                    the bucket's lookups by energy sub-bin (S sub-bins per bucket), writing the
//                    final slot order and q in slot order (the lookup kernel then streams q
//                    instead of gathering q_of[slot] at random)
//   k_bucket_gather  (split path) q in slot order without refining
// Order inside a bucket is whatever the shared-memory atomics give; results never depend
// on it (every lookup is independent and the hash is an integer sum).
#include <algorithm>
#include <cmath>
#include <cstdlib>

#include "lookup_common.cuh"

namespace xs {

constexpr int kSortTpb = 1024;
#ifndef XS_SCATTER_VEC
#define XS_SCATTER_VEC 1
#endif
#ifndef XS_SCATTER_ILP4
#define XS_SCATTER_ILP4 1
#endif
constexpr int64_t kScatterWindow = int64_t(64) << 20; // max bytes of slots one scatter launch writes
constexpr int64_t kScatterWindowLarge = int64_t(60) << 20; // slot arrays above 128 MB: 7 windows for 100M
#ifndef XS_SCATTER_ZERO
#define XS_SCATTER_ZERO 1
#endif
constexpr bool kScatterZero = XS_SCATTER_ZERO;
constexpr int64_t kZeroMinBytes = int64_t(96) << 20; // slot arrays above this get pre-zeroed windows

__global__ void __launch_bounds__(kSortTpb) k_bucket_count(SampleView sv, BucketPlan bp, int per_cta, Affine J_tpb,
                                                            uint32_t *__restrict__ hist, double *__restrict__ q_of,
                                                            uint16_t *__restrict__ key_of,
                                                            unsigned long long *__restrict__ ctl)
{
    pdl_wait();
    pdl_trigger();
    if (ctl && blockIdx.x == 0 && threadIdx.x == 0) { // the lookup kernel's work-queue counter
        ctl[0] = 0;                                 // and CTA-completion count (read only
        ctl[1] = 0;                                 // after this kernel)
    }
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
            if (q_of)
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
    pdl_wait();
    pdl_trigger();
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
// a block scan of the warp totals gives each warp its offset for the second pass.  Then, for
// the shard's buckets [kA, kB) (everything unsharded) whose slots are re-based to start at 0:
// base[K + m] = first slot of material m in the shard (clamped to [0, n]), base[K + 12] = n,
// the shard's lookups (also added to *n_acc), base[K + 13] = every bucket's total,
// base[K + 14] = base[kA] (the slot the shard's slots are re-based by).
__global__ void __launch_bounds__(1024) k_bucket_base(BucketPlan bp, int kA, int kB, uint32_t *__restrict__ base,
                                                      unsigned long long *__restrict__ n_acc)
{
    pdl_wait();
    pdl_trigger();
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
        const uint32_t total = wsum[31];
        const uint32_t s0 = kA < K ? base[kA] : total, s1 = kB < K ? base[kB] : total;
        const uint32_t n = s1 - s0;
        uint32_t mb[kMaterials];
#pragma unroll
        for (int m = 0; m < kMaterials; m++) {
            const uint32_t b = bp.kbase[m] < K ? base[bp.kbase[m]] : total;
            mb[m] = b <= s0 ? 0u : (b >= s1 ? n : b - s0);
        }
#pragma unroll
        for (int m = 0; m < kMaterials; m++)
            base[K + m] = mb[m];
        base[K + kMaterials] = n;
        base[K + kMaterials + 1] = total;
        base[K + kMaterials + 2] = s0;
        if (n_acc)
            atomicAdd(n_acc, (unsigned long long)n);
    }
}

// Writes the lookups whose key lies in [klo, khi) (one launch per window of buckets: the
// window's slots, ~kScatterWindow bytes, stay L2-resident while their random partial-sector
// writes merge; a slot array larger than L2 took DRAM read-modify-writes per 4 B store).
__global__ void __launch_bounds__(kSortTpb) k_bucket_scatter(int K, int klo, int khi, int per_cta, int count,
                                                              const uint32_t *__restrict__ hist,
                                                              const uint32_t *__restrict__ base,
                                                              const uint16_t *__restrict__ key_of,
                                                              uint32_t *__restrict__ slot_of)
{
    pdl_wait();
    pdl_trigger();
    extern __shared__ uint32_t sh[];
    const uint32_t *h = hist + (int64_t)blockIdx.x * K;
    const uint32_t rebase = base[K + kMaterials + 2]; // the shard's first slot (0 unsharded)
    for (int k = klo + threadIdx.x; k < khi; k += kSortTpb)
        sh[k] = base[k] + h[k] - rebase;
    __syncthreads();
    const int beg = blockIdx.x * per_cta;
    const int end = min(beg + per_cta, count);
    const uint32_t span = (uint32_t)(khi - klo);
    // 4 keys in flight per thread, then their shared-memory atomics and 4 B stores
    // (recording each lookup's rank in the count pass to drop the atomics was measured
    // slower)
#if XS_SCATTER_VEC
    // 8 keys per 16 B load (per_cta is a multiple of 8, so the chunk is 16 B aligned), two
    // loads in flight per thread; a thread's 8 lookups are consecutive offsets (any order
    // inside a bucket is valid)
    const int nvec = max(0, end - beg) >> 3;
    const uint4 *kv = reinterpret_cast<const uint4 *>(key_of + beg);
    auto put = [&](uint32_t w, int j0) {
        const uint32_t k0 = w & 0xffffu, k1 = w >> 16;
        if (k0 - (uint32_t)klo < span)
            slot_of[atomicAdd(&sh[k0], 1u)] = (uint32_t)j0;
        if (k1 - (uint32_t)klo < span)
            slot_of[atomicAdd(&sh[k1], 1u)] = (uint32_t)(j0 + 1);
    };
    int v = threadIdx.x;
#if XS_SCATTER_ILP4
    // four 16 B key loads in flight per thread (the window's keys are a sparse 1/nwin of the
    // stream: the kernel waits on these loads, ncu long_scoreboard 54%)
    for (; v + 3 * kSortTpb < nvec; v += 4 * kSortTpb) {
        const uint4 a = __ldg(kv + v), b = __ldg(kv + v + kSortTpb);
        const uint4 c = __ldg(kv + v + 2 * kSortTpb), d = __ldg(kv + v + 3 * kSortTpb);
        const int ja = beg + 8 * v, jb = ja + 8 * kSortTpb, jc = jb + 8 * kSortTpb, jd = jc + 8 * kSortTpb;
        put(a.x, ja); put(a.y, ja + 2); put(a.z, ja + 4); put(a.w, ja + 6);
        put(b.x, jb); put(b.y, jb + 2); put(b.z, jb + 4); put(b.w, jb + 6);
        put(c.x, jc); put(c.y, jc + 2); put(c.z, jc + 4); put(c.w, jc + 6);
        put(d.x, jd); put(d.y, jd + 2); put(d.z, jd + 4); put(d.w, jd + 6);
    }
#endif
    for (; v + kSortTpb < nvec; v += 2 * kSortTpb) {
        const uint4 a = __ldg(kv + v), b = __ldg(kv + v + kSortTpb);
        const int ja = beg + 8 * v, jb = ja + 8 * kSortTpb;
        put(a.x, ja); put(a.y, ja + 2); put(a.z, ja + 4); put(a.w, ja + 6);
        put(b.x, jb); put(b.y, jb + 2); put(b.z, jb + 4); put(b.w, jb + 6);
    }
    for (; v < nvec; v += kSortTpb) {
        const uint4 a = __ldg(kv + v);
        const int ja = beg + 8 * v;
        put(a.x, ja); put(a.y, ja + 2); put(a.z, ja + 4); put(a.w, ja + 6);
    }
    for (int j = beg + 8 * nvec + threadIdx.x; j < end; j += kSortTpb) {
        const uint32_t k = key_of[j];
        if (k - (uint32_t)klo < span)
            slot_of[atomicAdd(&sh[k], 1u)] = (uint32_t)j;
    }
#else
    int j = beg + threadIdx.x;
    for (; j + 3 * kSortTpb < end; j += 4 * kSortTpb) {
        uint32_t kk[4];
#pragma unroll
        for (int u = 0; u < 4; u++)
            kk[u] = key_of[j + u * kSortTpb];
#pragma unroll
        for (int u = 0; u < 4; u++)
            if (kk[u] - (uint32_t)klo < span)
                slot_of[atomicAdd(&sh[kk[u]], 1u)] = (uint32_t)(j + u * kSortTpb);
    }
    for (; j < end; j += kSortTpb) {
        const uint32_t k = key_of[j];
        if (k - (uint32_t)klo < span)
            slot_of[atomicAdd(&sh[k], 1u)] = (uint32_t)j;
    }
#endif
}

// Zero the slots [base[klo], base[khi]) of the next scatter window with whole 16 B stores: the
// L2 then holds the window's lines before the scatter's 4 B writes arrive, instead of reading
// every sector from DRAM on its first partial write (the scatter's DRAM reads were ~the
// window's size on top of the keys)
__global__ void __launch_bounds__(1024) k_zero_window(int K, int klo, int khi, int count,
                                                      const uint32_t *__restrict__ base, uint32_t *__restrict__ slot_of)
{
    pdl_wait();
    pdl_trigger();
    const uint32_t rebase = base[K + kMaterials + 2], total = base[K + kMaterials + 1];
    const uint32_t s0 = base[klo] - rebase, s1 = (khi < K ? base[khi] : total) - rebase;
    (void)count;
    const uint32_t a0 = (s0 + 3) & ~3u, a1 = s1 & ~3u; // 16 B aligned body
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (a0 < a1) {
        uint4 *p = reinterpret_cast<uint4 *>(slot_of + a0);
        const int64_t nv = (a1 - a0) >> 2;
        for (int64_t i = t0; i < nv; i += stride)
            p[i] = make_uint4(0, 0, 0, 0);
    }
    if (t0 < 8) { // the unaligned head and tail slots
        const uint32_t j = t0 < 4 ? s0 + (uint32_t)t0 : a1 + (uint32_t)(t0 - 4);
        if (t0 < 4 ? j < min(a0, s1) : (j >= max(a1, s0) && j < s1))
            slot_of[j] = 0;
    }
}

__global__ void k_bucket_gather(int count, const uint32_t *__restrict__ slot_of, const double *__restrict__ q_of,
                                double *__restrict__ q_sorted)
{
    for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < count; j += gridDim.x * blockDim.x)
        q_sorted[j] = __ldg(q_of + __ldg(slot_of + j));
}

// k_bucket_refine: work group g owns the buckets [g B, g B + B) (under the refine plan every
// bucket holds ~count/K lookups, so B buckets are ~kRefineTarget lookups), i.e. the slots
// [base[g B], base[g B + B]); a persistent grid of CTAs takes the groups in turn.  Bucket k
// of material m covers energies [b / nb[m], (b + 1) / nb[m]) (b = k - kbase[m]); it is cut
// into S sub-bins, sub = floor((q nb[m] - b) S) clamped to [0, S), and the CTA
// counting-sorts the group's slots by (bucket, sub-bin): histogram in shared memory, block
// scan, the refined order assembled in shared memory, then written out coalesced (scattered
// stores are L2-request bound).  The energy of lookup offset j is recomputed, not gathered:
// its stream state is J(2 j) s_base with s_base = J(2 first) seed (one Listing-7 jump per
// chunk, on the host), and J(2 j) is the product of the byte maps J(2 d 256^t), d = byte t
// of j (tables in shared memory; affine maps of one LCG commute, and arithmetic mod 2^64 maps
// onto mod 2^63, so this is exactly sample_lookup's state).  A group larger than kRefineCap
// (a pathological bucket) is handled by re-reading its slots, with scattered stores.  Any
// order is a valid ordering (results never depend on it): the sub-bin function needs no
// exact monotonicity, and the order inside a sub-bin is whatever the atomics give.
constexpr int kRefineTpb = 256;
#ifndef XS_REFINE_PER
#define XS_REFINE_PER 12
#endif
#ifndef XS_REFINE_MINB
#define XS_REFINE_MINB 3
#endif
constexpr int kRefinePer = XS_REFINE_PER;           // slots per thread in registers
constexpr int kRefineCap = kRefineTpb * kRefinePer; // 3072 slots per group
#ifndef XS_REFINE_BINS
#define XS_REFINE_BINS 1024
#endif
constexpr int kRefineBins = XS_REFINE_BINS;         // B x S
constexpr int kRefineTarget = kRefineCap * 5 / 8;   // mean slots per group the plan aims at
static_assert(kRefineBins < 2048 && kRefineCap < (1 << 21), "bin and rank are packed into 11 + 21 bits");
constexpr int kRefineMaxB = 64;
// jump tables for lookup offsets j < 2^28 (kChunkSorted): digit t of j (widths 10, 9, 9 bits)
// indexes table t, J(2 d 2^(shift t)); three table maps per energy instead of four byte maps
// (and no padding slots, below: refine 1.09 -> 0.94 ms on large-U)
constexpr int kJumpDigits = 3;
__host__ __device__ constexpr int jump_bits(int t) { return t == 0 ? 10 : 9; }
__host__ __device__ constexpr int jump_shift(int t) { return t == 0 ? 0 : (t == 1 ? 10 : 19); }
__host__ __device__ constexpr int jump_base(int t) { return t == 0 ? 0 : (t == 1 ? 1024 : 1536); }
constexpr int kJumpEntries = 2048;
static_assert(jump_shift(2) + jump_bits(2) == 28, "the tables cover offsets < 2^28");

// sub-bin of a lookup from its 63-bit stream state u (q = RN(u) 2^-63): the integer form of
// floor((q nb - b) S), v = (u >> 20) nb ~ q nb 2^43 (< 2^59); rounding at the bucket edges
// only moves a lookup into the edge sub-bin (clamped)
__device__ __forceinline__ int refine_bin(uint64_t u, uint32_t nb, int b, int kb, int s_log2)
{
    const uint64_t v = (u >> 20) * (uint64_t)nb;
    int t = (int)(v >> (43 - s_log2)) - (b << s_log2);
    const int S = 1 << s_log2;
    t = t < 0 ? 0 : (t > S - 1 ? S - 1 : t);
    return (kb << s_log2) + t;
}

// stream state of lookup offset j (< 2^28) after its energy draw (sample_lookup: q = RN(u)
// 2^-63): the digit maps applied to the chunk's base state one after the other (a digit of 0
// maps through the identity)
__device__ __forceinline__ uint64_t energy_state(const Affine *jt, uint64_t s, uint32_t j)
{
#pragma unroll
    for (int t = 0; t < kJumpDigits; t++) {
        const Affine m = jt[jump_base(t) + ((j >> jump_shift(t)) & ((1u << jump_bits(t)) - 1))];
        s = m.a * s + m.c;
    }
    return lcg_step(s & kMod63);
}

__global__ void __launch_bounds__(kRefineTpb, XS_REFINE_MINB) k_bucket_refine(BucketPlan bp, int kA, int kB, int B,
                                                                  int s_log2,
                                                                  uint64_t s_base, const Affine *__restrict__ jt_g,
                                                                  const uint32_t *__restrict__ base,
                                                                  const uint32_t *__restrict__ slot_in,
                                                                  uint32_t *__restrict__ slot_out,
                                                                  double *__restrict__ q_out)
{
    pdl_wait();
    pdl_trigger();
    __shared__ Affine s_jt[kJumpEntries];
    __shared__ uint32_t s_hist[kRefineBins];
    __shared__ uint32_t s_bs[kRefineMaxB + 1]; // slot bounds of the group's buckets
    __shared__ uint32_t s_nbm[kRefineMaxB];
    __shared__ int s_b[kRefineMaxB];
    __shared__ uint32_t s_wsum[kRefineTpb / 32];
    extern __shared__ __align__(16) unsigned char s_stage[]; // the refined order: [cap] q, then [cap] offsets
    double *s_q = reinterpret_cast<double *>(s_stage);
    uint32_t *s_r = reinterpret_cast<uint32_t *>(s_q + kRefineCap);
    const int K = bp.K;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    for (int i = tid; i < kJumpEntries; i += kRefineTpb)
        s_jt[i] = jt_g[i];
    const int ngroups = (kB - kA + B - 1) / B;
    // the shard's slots start at 0 (base[K + 14] = base[kA]; 0 and kA = 0 unsharded)
    const uint32_t rebase = __ldg(base + K + kMaterials + 2), total = __ldg(base + K + kMaterials + 1);
    for (int grp = blockIdx.x; grp < ngroups; grp += gridDim.x) {
        const int k0 = kA + grp * B, nbk = min(B, kB - k0);
        if (tid <= nbk)
            s_bs[tid] = ((k0 + tid < K) ? __ldg(base + k0 + tid) : total) - rebase;
        if (tid < nbk) {
            const int k = k0 + tid;
            int m = 0;
#pragma unroll
            for (int mm = 1; mm < kMaterials; mm++)
                m += (k >= bp.kbase[mm]) ? 1 : 0;
            s_nbm[tid] = (uint32_t)bp.nb[m];
            s_b[tid] = k - bp.kbase[m];
        }
        const int nbins = nbk << s_log2;
        for (int i = tid; i < nbins; i += kRefineTpb)
            s_hist[i] = 0u;
        __syncthreads();
        const uint32_t s0 = s_bs[0], s1 = s_bs[nbk];
        const bool regs = s1 - s0 <= (uint32_t)kRefineCap; // CTA-uniform
        // slots t of a thread increase, so their bucket kb (the last with s_bs[kb] <= t) is
        // found by walking forward from the previous one
        int kb = 0;
        auto bin_of = [&](uint32_t t, uint64_t u) {
            while (kb + 1 < nbk && s_bs[kb + 1] <= t)
                kb++;
            return refine_bin(u, s_nbm[kb], s_b[kb], kb, s_log2);
        };
        uint32_t r[kRefinePer];
        double q[kRefinePer];
        int bin[kRefinePer];
        if (regs) {
            // positions past the group (the group holds ~2/3 of kRefineCap on average) skip the
            // energy, bin and atomic: slot u of a warp's lanes is 32 consecutive positions, so
            // the branch is warp-uniform except in one warp
#pragma unroll
            for (int u = 0; u < kRefinePer; u++) {
                const uint32_t t = s0 + tid + u * kRefineTpb;
                r[u] = t < s1 ? __ldg(slot_in + t) : 0u;
            }
#pragma unroll
            for (int u = 0; u < kRefinePer; u++) {
                const uint32_t t = s0 + tid + u * kRefineTpb;
                if (t < s1) {
                    const uint64_t st = energy_state(s_jt, s_base, r[u]);
                    q[u] = u63_to_double(st);
                    const int b = bin_of(t, st);
                    // the slot's rank inside its bin from the histogram atomic itself, packed
                    // above the bin index (bin < 2^11, rank < kRefineCap < 2^21): the placement
                    // below needs no second atomic (sort 0.406 -> 0.384 ms small, 2.47 -> 2.41
                    // large-U)
                    bin[u] = b | (int)(atomicAdd(&s_hist[b], 1u) << 11);
                } else {
                    q[u] = 0.0;
                    bin[u] = -1;
                }
            }
        } else {
            for (uint32_t t = s0 + tid; t < s1; t += kRefineTpb)
                atomicAdd(&s_hist[bin_of(t, energy_state(s_jt, s_base, __ldg(slot_in + t)))], 1u);
        }
        __syncthreads();
        // exclusive scan of s_hist[0 .. nbins): warp w owns kRows rows of 32 bins (lane =
        // column: no bank conflicts)
        constexpr int kRows = kRefineBins >= kRefineTpb ? kRefineBins / kRefineTpb : 1;
        const int wb = wid * 32 * kRows;
        uint32_t wsum = 0;
#pragma unroll
        for (int i = 0; i < kRows; i++) {
            const int k = wb + i * 32 + lane;
            wsum += k < nbins ? s_hist[k] : 0u;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
            wsum += __shfl_xor_sync(0xffffffffu, wsum, o);
        if (lane == 0)
            s_wsum[wid] = wsum;
        __syncthreads();
        uint32_t carry = 0;
        for (int w = 0; w < wid; w++)
            carry += s_wsum[w];
#pragma unroll
        for (int i = 0; i < kRows; i++) {
            const int k = wb + i * 32 + lane;
            const uint32_t x = k < nbins ? s_hist[k] : 0u;
            uint32_t incl = x;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                incl += (lane >= o) ? y : 0u;
            }
            if (k < nbins)
                s_hist[k] = carry + incl - x;
            carry += __shfl_sync(0xffffffffu, incl, 31);
        }
        __syncthreads();
        if (regs) {
#pragma unroll
            for (int u = 0; u < kRefinePer; u++) {
                if (bin[u] >= 0) {
                    const uint32_t pos = s_hist[bin[u] & 2047] + ((uint32_t)bin[u] >> 11);
                    s_r[pos] = r[u];
                    s_q[pos] = q[u];
                }
            }
            __syncthreads();
            const uint32_t n = s1 - s0;
            for (uint32_t i = tid; i < n; i += kRefineTpb) {
                slot_out[s0 + i] = s_r[i];
                q_out[s0 + i] = s_q[i];
            }
        } else {
            kb = 0;
            for (uint32_t t = s0 + tid; t < s1; t += kRefineTpb) {
                const uint32_t rr = __ldg(slot_in + t);
                const uint64_t st = energy_state(s_jt, s_base, rr);
                const double qq = u63_to_double(st);
                const uint32_t pos = s0 + atomicAdd(&s_hist[bin_of(t, st)], 1u);
                slot_out[pos] = rr;
                q_out[pos] = qq;
            }
        }
        __syncthreads(); // the group's shared state is done before the next group's
    }
}

static int sm_count_dev() { return sm_count_cached(); }

static void ensure_sort_space(Grid &g, int64_t chunk, int ctas, int K)
{
    if (g.cap < chunk) {
        cudaFree(g.sq);
        cudaFree(g.si);
        cudaFree(g.skey);
        cudaFree(g.qs);
        cudaFree(g.si2);
        g.sq = g.qs = nullptr;
        g.si = g.si2 = nullptr;
        g.skey = nullptr;
        g.cap = 0;
        XS_CUDA_TRY(cudaMalloc(&g.sq, (size_t)chunk * sizeof(double)));
        XS_CUDA_TRY(cudaMalloc(&g.qs, (size_t)chunk * sizeof(double)));
        XS_CUDA_TRY(cudaMalloc(&g.si, (size_t)chunk * sizeof(uint32_t)));
        XS_CUDA_TRY(cudaMalloc(&g.si2, (size_t)chunk * sizeof(uint32_t)));
        XS_CUDA_TRY(cudaMalloc(&g.skey, (size_t)chunk * sizeof(uint16_t)));
        g.cap = chunk;
    }
    if (!g.jt) { // digit jump tables of k_bucket_refine: jt[base t + d] = J(2 d 2^(shift t))
        static Affine h[kJumpEntries];
        for (int t = 0; t < kJumpDigits; t++)
            for (int d = 0; d < (1 << jump_bits(t)); d++)
                h[jump_base(t) + d] = lcg_jump(2 * ((uint64_t)d << jump_shift(t)));
        XS_CUDA_TRY(cudaMalloc(&g.jt, sizeof(h)));
        XS_CUDA_TRY(cudaMemcpy(g.jt, h, sizeof(h), cudaMemcpyHostToDevice));
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

static BucketPlan make_plan(const Grid &g, int total, bool by_lookups)
{
    BucketPlan bp{};
    double w[kMaterials], W = 0;
    for (int m = 0; m < kMaterials; m++) {
        const double p = (m == 0) ? 1.0 - g.thresholds[11] : g.thresholds[m] - g.thresholds[m - 1];
        w[m] = by_lookups ? p : p * g.num_nucs[m];
        W += w[m];
    }
    // floor(total * share) + at most one bump to 1 per material stays <= total + 12
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

// Key-range shard boundaries: shard s of n owns buckets [b(s), b(s+1)), b(s) the first bucket at
// which the expected cost of the buckets before it reaches s/n of the total -- a bucket's
// expected cost is its expected lookups (P(m) / nb[m] of the range) times (num_nucs[m] +
// kShardLookupCost), so the fuel's buckets (81% of large's pairs in 14% of its lookups) are
// spread over most shards.  Monotone in s, b(0) = 0, b(n) = K: the shards partition the buckets.
#ifndef XS_SHARD_LOOKUP_COST
#define XS_SHARD_LOOKUP_COST 22
#endif
constexpr double kShardLookupCost = XS_SHARD_LOOKUP_COST;

static int shard_boundary(const Grid &g, const BucketPlan &bp, int s, int n)
{
    if (s <= 0)
        return 0;
    if (s >= n)
        return bp.K;
    double w[kMaterials], W = 0;
    for (int m = 0; m < kMaterials; m++) {
        const double p = (m == 0) ? 1.0 - g.thresholds[11] : g.thresholds[m] - g.thresholds[m - 1];
        // expected cost of the material, spread evenly over its buckets: its pairs plus a
        // per-lookup share (the sort's scatter and refine, the lookup kernel's per-warp window
        // and staging work) worth ~kShardLookupCost pairs
        w[m] = p * (g.num_nucs[m] + kShardLookupCost);
        W += w[m];
    }
    const double target = W * s / n;
    double cum = 0;
    for (int m = 0; m < kMaterials; m++) {
        if (cum + w[m] >= target && w[m] > 0) {
            const int k = bp.kbase[m] + (int)std::ceil((target - cum) / (w[m] / bp.nb[m]) - 1e-9);
            return std::min(std::max(k, bp.kbase[m]), bp.kbase[m + 1]);
        }
        cum += w[m];
    }
    return bp.K;
}

int launch_bucket_sort(Grid &g, const SampleView &sv, int nb_avg, int post, cudaStream_t stream, int *K_out,
                       int shard, int nshards, unsigned long long *n_acc)
{
    {
        const int bytes = kMaterials * kMaxEnergyBins * 4; // the largest histogram a plan can ask for
        resident_ctas((const void *)k_bucket_count, kSortTpb, bytes);
        resident_ctas((const void *)k_bucket_scatter, kSortTpb, bytes);
    }
    const int64_t cn = sv.count;
    // refine: buckets of equal expected size (the sub-bins give every material its energy
    // resolution); coarse: cost-weighted, the material that dominates the pairs gets the
    // finest buckets
    const bool refine = post == kSortPostRefine && nb_avg > 1;
    // coarse: 12 (nb_avg - 1) buckets; refine: one bucket per ~kRefineTarget lookups (a
    // refine group is then one bucket), at most the coarse count
    const int total_coarse = nb_avg > 1 ? kMaterials * (nb_avg - 1) : 0;
    const int total = refine ? (int)std::min<int64_t>(total_coarse, std::max<int64_t>(kMaterials, cn / kRefineTarget))
                             : total_coarse;
    const BucketPlan bp = make_plan(g, total, refine);
    const int K = bp.K;
    *K_out = K;
    const int sms = sm_count_dev();
    const int ctas = (int)std::max<int64_t>(1, std::min<int64_t>(sms, (cn + kSortTpb - 1) / kSortTpb));
    const int per_cta = (int)(((cn + ctas - 1) / ctas + 7) / 8 * 8); // 16 B aligned key chunks
    ensure_sort_space(g, cn, ctas, K);
    const Affine J = lcg_jump(2 * (uint64_t)kSortTpb);
    const size_t smem = (size_t)K * 4;
    // refine recomputes energies from lookup offsets: no q_of
    launch_pdl(k_bucket_count, ctas, kSortTpb, (int)smem, stream, sv, bp, per_cta, J, g.hist,
               refine ? nullptr : g.sq, g.skey, (unsigned long long *)(g.stats_d + 4));
    launch_pdl(k_bucket_colscan, (K + 31) / 32, 32 * kColWarps, 0, stream, K, ctas, g.hist, g.base);
    // key-range shard (xs_opts.shard_*): buckets [kA, kB) -- every lookup is drawn and counted,
    // only the shard's are ordered (slots re-based to start at 0 by k_bucket_base)
    const int kA = shard_boundary(g, bp, shard, nshards), kB = shard_boundary(g, bp, shard + 1, nshards);
    const int64_t cn_own = (cn * (kB - kA) + K - 1) / K; // expected slots of the shard
    launch_pdl(k_bucket_base, 1, 1024, 0, stream, bp, kA, kB, g.base, n_acc);
    // windows of ~equal expected slot counts (refine: equal-size buckets; coarse: cost-weighted
    // buckets, so the windows are only approximately equal)
    // window: 1/6 of the slot array, at least 16 MB, and 60 MiB once the slots exceed 128 MB --
    // more windows keep each one's random writes more L2-local, but every window re-reads all
    // 2 B keys (measured, sort ms with pre-zeroing: 25M lookups 16 MB 0.558 / 64 MB 0.613;
    // 50M: 6 windows 1.285, 5 1.142, 3 1.126; 100M: 9 windows 1.815, 7 1.80, 6 1.88-1.91;
    // 125M: 11 windows 2.32, 8 2.25 -- profiles/r02n_mid2.jsonl, r02g13_winsweep.jsonl)
    int64_t win_bytes = cn_own * 4 > (int64_t(128) << 20)
                            ? kScatterWindowLarge
                            : std::min<int64_t>(kScatterWindow, std::max<int64_t>(int64_t(16) << 20, cn_own * 4 / 6));
    if (const char *env = std::getenv("XS_SCATTER_WINDOW_MB"))
        win_bytes = std::max(1ll, std::atoll(env)) << 20;
    int nwin = (int)std::max<int64_t>(1, std::min<int64_t>(kB - kA, (cn_own * 4 + win_bytes - 1) / win_bytes));
    if (const char *env = std::getenv("XS_TEST_SCATTER_WINDOWS")) // test hook: force the window count
        nwin = (int)std::max<int64_t>(1, std::min<int64_t>(kB - kA, std::atoll(env)));
    // pre-zero each window when the slot array exceeds the L2 (large-U / XL sort 2.16 / 2.76 ->
    // 1.82 / 2.25 ms); an L2-sized one (17M lookups: 68 MB) is resident already and zeroing
    // only adds work (small 0.337 -> 0.385 ms)
    const bool zero = kScatterZero && (cn_own * 4 > kZeroMinBytes || std::getenv("XS_TEST_SCATTER_ZERO"));
    for (int w = 0; w < nwin; w++) {
        const int klo = kA + (int)((int64_t)(kB - kA) * w / nwin), khi = kA + (int)((int64_t)(kB - kA) * (w + 1) / nwin);
        if (zero)
            launch_pdl(k_zero_window, sms * 2, 1024, 0, stream, K, klo, khi, (int)cn, (const uint32_t *)g.base,
                       refine ? g.si2 : g.si);
        launch_pdl(k_bucket_scatter, ctas, kSortTpb, (int)smem, stream, K, klo, khi, per_cta, (int)cn, g.hist, g.base,
                   g.skey, refine ? g.si2 : g.si);
    }
    XS_CUDA_TRY(cudaGetLastError());
    if (refine) {
        const double avg = (double)cn / K; // lookups per bucket (sharded or not)
        const int B = (int)std::max(1.0, std::min<double>(kRefineMaxB, kRefineTarget / std::max(avg, 1.0)));
        int s_log2 = 0;
        while ((B << (s_log2 + 1)) <= kRefineBins)
            s_log2++;
        const int rsmem = kRefineCap * 12;
        const int per_sm = resident_ctas((const void *)k_bucket_refine, kRefineTpb, rsmem);
        const int ngroups = (kB - kA + B - 1) / B;
        const int rblocks = std::max(1, std::min(ngroups, sms * std::max(per_sm, 1)));
        launch_pdl(k_bucket_refine, rblocks, kRefineTpb, rsmem, stream, bp, kA, kB, B, s_log2,
                   lcg_apply(lcg_jump(2 * (uint64_t)sv.first), sv.seed), (const Affine *)g.jt,
                   (const uint32_t *)g.base, (const uint32_t *)g.si2, g.si, g.qs);
        XS_CUDA_TRY(cudaGetLastError());
        return 4 + nwin * (zero ? 2 : 1);
    }
    if (post != kSortPostGather)
        return 3 + nwin * (zero ? 2 : 1);
    const int gblocks = (int)std::min<int64_t>((cn + 255) / 256, (int64_t)sms * 8);
    k_bucket_gather<<<gblocks, 256, 0, stream>>>((int)cn, g.si, g.sq, g.qs);
    XS_CUDA_TRY(cudaGetLastError());
    return 4 + nwin * (zero ? 2 : 1);
}

} // namespace xs
