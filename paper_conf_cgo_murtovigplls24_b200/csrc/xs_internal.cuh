// xs_internal.cuh -- grid object, error plumbing and kernel-argument structs of libxs.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <string>

#include "../../include/xs.h"
#include "rng.cuh"

namespace xs {

// ---- errors --------------------------------------------------------------------------
struct Error {
    int code;
    std::string msg;
};
void set_error(int code, const std::string &msg);
void clear_error();

#define XS_CUDA_TRY(expr)                                                                       \
    do {                                                                                        \
        cudaError_t e_ = (expr);                                                                \
        if (e_ != cudaSuccess)                                                                  \
            throw ::xs::Error{e_ == cudaErrorMemoryAllocation ? XS_ENOMEM : XS_ECUDA,           \
                              std::string(#expr) + ": " + cudaGetErrorString(e_)};              \
    } while (0)

#define XS_CHECK_ARG(cond, what)                                                                \
    do {                                                                                        \
        if (!(cond))                                                                            \
            throw ::xs::Error{XS_EINVAL, what};                                                 \
    } while (0)

constexpr int kMaterials = 12;
constexpr int kMaxEnergyBins = 4096;
#ifndef XS_IV
#define XS_IV 0
#endif
// XS_IV: lookups interpolate from per-interval records (iv) instead of point pairs (pts)
constexpr bool kIv = XS_IV;
#ifndef XS_S_TMA
#define XS_S_TMA 1
#endif
constexpr bool kTmaStage = XS_S_TMA; // XS_SEARCH_S stages interval records with cp.async.bulk
#ifndef XS_HASH_FAST
#define XS_HASH_FAST 1
#endif
// XS_HASH_FAST: H and S find the hash-grid window with a multiply and overlapped guard loads
// (lookup_common.cuh lower_index; 0 = R7 as written, for the A/B)
constexpr bool kHashFast = XS_HASH_FAST;
#ifndef XS_HASH_K4
#define XS_HASH_K4 1
#endif
// XS_HASH_K4: that window searched 4-ary (search.cuh search_K4); 0 = Listing 1 (M)
constexpr bool kHashK4 = XS_HASH_K4;
#ifndef XS_BIN_K4
#define XS_BIN_K4 1
#endif
// XS_BIN_K4: the bin windows of H and S (nuclide and unionized grids) searched 4-ary too; 0 = U2
constexpr bool kBinK4 = XS_BIN_K4;
constexpr int kTreeFan = 16;     // separator keys per node: one 128 B line
constexpr int kTreeMaxLevels = 6; // n < 17^6 * 16 for every n_gridpoints < 2^31

// ---- the grid in HBM -----------------------------------------------------
//   E   [n_nuc][n]      fp64  search keys, SoA (8 B stride: the probes of Listing 1)
//   pts [n_nuc][n][6]   fp64  {E, total, elastic, absorption, fission, nu-fission}: one
//                             48 B record per point, three 16 B vector loads
//   U   [N]             fp64  unionized energies (grid_type 0)
//   IDX [N][n_nuc]      int32 unionized lower indices (grid_type 0)
//   H   [bins][n_nuc]   int32 hash-bin lower indices (grid_type 2)
//   mats [12][max] int32, concs [12][max] fp64, num_nucs [12] int32
struct Grid {
    int device = 0;
    int64_t n_nuc = 0, n = 0, N = 0, bins = 0;
    int grid_type = 1;
    uint64_t seed = 0;
    int32_t max_nucs = 0;
    int32_t num_nucs[kMaterials] = {};
    double thresholds[kMaterials] = {}; // pick_mat running sums T[m]
    uint64_t device_bytes = 0;

    double *E = nullptr;
    double *pts = nullptr;
    // iv [n_nuc][n-1][12]: interval L's record {E[L+1], E[L+1]-E[L], (X_c[L+1],
    // X_c[L+1]-X_c[L]) for c = 0..4} -- the differences the interpolation needs, rounded
    // once at build time exactly as the lookup would round them (XS_IV)
    double *iv = nullptr;
    // ivs [n_nuc][n-1][14] (XS_S_TMA): the staged kernel's 112 B interval record
    // {E_hi, 0, d = E_hi - E_lo, RN(1/d), (X_c,hi, X_c,hi - X_c,lo) x 5}, copied into shared
    // memory by the bulk-copy engine (cp.async.bulk) instead of assembled by the warp
    double *ivs = nullptr;
    // separator tree of every nuclide row (XS_SEARCH_W): level d has
    // 17^d nodes of 16 keys; node keys are E at base + (t+1)*stride[d] (+inf past n)
    double *tkeys = nullptr;
    int32_t t_levels = 0;
    int32_t t_stride[kTreeMaxLevels] = {};
    int32_t t_off[kTreeMaxLevels] = {};
    int32_t t_leaf = 0;       // elements probed at the leaf (<= 16)
    int64_t t_per_nuc = 0;    // keys per nuclide
    // bin table of every nuclide row (XS_SEARCH_H): [n_nuc][2^b_log2]
    struct BinEntry *bnd = nullptr;
    int32_t b_log2 = 0;
    // bin table of the unionized energies (XS_SEARCH_H on XS_UNIONIZED): [2^u_log2]
    struct BinEntry *ubnd = nullptr;
    int32_t u_log2 = 0;
    double *U = nullptr;
    int32_t *IDX = nullptr;
    int32_t *H = nullptr;
    int32_t *mats = nullptr;
    double *concs = nullptr;
    int32_t *num_nucs_d = nullptr;
    void *refs = nullptr;            // NucRef [12][max_nucs]: row pointers + conc per (mat, j)

    // per-grid scratch (grown on demand; calls on one grid are serialised by the caller)
    uint64_t *stats_d = nullptr;     // [8] hash, pairs, work counter
    uint64_t *stats_h = nullptr;     // pinned mirror
    double *sq = nullptr;            // energies by lookup offset (coalesced writes) [cap]
    uint32_t *si = nullptr;          // lookup offsets in (material, energy) order  [cap]
    uint16_t *skey = nullptr;        // bucket key by lookup offset                [cap]
    double *qs = nullptr;            // energies in (material, energy) order       [cap]
    Affine *jt = nullptr;            // refine: digit jump tables (sort.cu energy_state)
    uint32_t *si2 = nullptr;         // refine: the coarse slot order before k_bucket_refine [cap]
    int32_t *Lbuf = nullptr;         // split path: lower index of every pair      [lcap]
    int64_t lcap = 0;
    uint32_t *mb_h = nullptr;        // pinned: material bases of the last sort
    uint32_t *hist = nullptr;        // per-CTA bucket histograms [ctas][K]
    uint32_t *base = nullptr;        // [K + 16]: bucket bases, then material bases
    int64_t cap = 0, hist_cap = 0;
    double *stage = nullptr;         // device staging for host outputs: 2 buffers
    int64_t stage_cap = 0;
    cudaStream_t copy_stream = nullptr; // D2H of staged outputs, overlapped with compute
    cudaEvent_t ev_done[2] = {}, ev_copied[2] = {};
    cudaEvent_t ev[8] = {};
};

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev)
    {
        cudaGetDevice(&prev);
        if (prev != dev)
            cudaSetDevice(dev);
    }
    ~DeviceGuard()
    {
        if (prev >= 0)
            cudaSetDevice(prev);
    }
};

// ---- kernel arguments ----------------------------------------------------------------
// One bin b of a sorted row A (XS_SEARCH_H): lo = L(b/2^k), cnt = L((b+1)/2^k) - lo,
// e_next = A[lo + 1] -- for cnt <= 1 the lower index of any q in the bin is
// lo + (cnt && e_next <= q) without touching the row.
struct alignas(16) BinEntry {
    int32_t lo;
    int32_t cnt;
    double e_next;
};
// Everything the lookup loop needs about nuclide j of material m, precomputed at grid
// creation so the loop does one 32 B broadcast load instead of 64-bit row arithmetic.
struct NucRef {
    const double *E;   // energy row of the nuclide            (E + nuc * n)
    const double *pts; // interpolation records: pts + nuc*n*6 (48 B points) or, with XS_IV,
                       // iv + nuc*(n-1)*12 (96 B intervals)
    const double *T;   // separator tree of the nuclide, or NULL
    const BinEntry *B; // bin table of the nuclide, or NULL
    double conc;       // concs[m][j]
    int64_t nuc;       // nuclide id
};

struct GridView {
    const double *__restrict__ E;
    const double *__restrict__ pts;
    const double *__restrict__ iv;
    const double *__restrict__ ivs;
    const double *__restrict__ U;
    const int32_t *__restrict__ IDX;
    const int32_t *__restrict__ H;
    const int32_t *__restrict__ mats;
    const double *__restrict__ concs;
    const int32_t *__restrict__ num_nucs;
    const NucRef *__restrict__ refs;
    int32_t n;        // gridpoints per nuclide
    int32_t n_nuc;
    int32_t N;        // n_nuc * n
    int32_t bins;
    int32_t max_nucs;
    int32_t t_levels;
    double du;        // 1.0 / bins
    const double *__restrict__ tkeys;
    int32_t t_stride[kTreeMaxLevels];
    int32_t t_off[kTreeMaxLevels];
    int32_t t_leaf;
    int32_t t_per_nuc;
    int32_t b_log2;   // XS_SEARCH_H bins = 2^b_log2 (0: no table)
    int32_t u_log2;   // unionized XS_SEARCH_H bins = 2^u_log2 (0: no table)
    const BinEntry *__restrict__ bnd;
    const BinEntry *__restrict__ ubnd;
};

struct SampleView {
    uint64_t seed;
    int64_t first;
    int64_t count;
    double T[kMaterials]; // pick_mat thresholds, T[0] unused
};

GridView make_view(const Grid &g);
SampleView make_sample_view(const Grid &g, uint64_t seed, int64_t first, int64_t count);

// Lookups of one chunk in (material, energy) order.
struct SortedView {
    const double *__restrict__ q;        // energy of sorted slot j (split path, refined sort), else null
    const double *__restrict__ q_of;     // energy by lookup offset
    const uint32_t *__restrict__ slot;   // lookup offset (i - first) of sorted slot j
    const uint32_t *__restrict__ mb_dev; // device copy of matbase (fused path)
    int *work;                           // fused path: work-chunk counter (zeroed per chunk)
    unsigned int *done;                  // S, last chunk: CTAs finished (zeroed with work)
    unsigned long long *pub;             // S, last chunk: host-mapped {hash, pairs, lookups}
                                         // written by the last CTA (no device-to-host copy), else null
    const uint32_t *count_dev;           // S: the slots to process (base[K + 12]: the shard's
                                         // lookups), else null (sv.count)
    uint32_t matbase[kMaterials + 1];    // split path: first slot of each material; [12] = count
};

// Pair buffer of the split path: material m's pairs start at pairbase[m], laid out
// nuclide-major ([jn][j - matbase[m]]) so a warp's stores and loads coalesce.
struct PairView {
    int32_t *__restrict__ L;
    uint64_t pairbase[kMaterials];
};

// grid.cu
void build_grid(Grid &g);
void free_grid(Grid &g);
uint64_t grid_checksum(const Grid &g);

// sort.cu: the (material, energy) counting sort of one chunk with `nb_avg` energy buckets
// per material on average; leaves g.sq (energy by lookup offset) and g.si (slot -> offset)
// filled and the material bases at g.base + *K_out (device).  Returns the kernels launched.
// post = kSortPostNone, kSortPostGather (g.qs = q in slot order) or kSortPostRefine
// (k_bucket_refine: every bucket re-ordered by energy sub-bin, g.si and g.qs rewritten).
enum { kSortPostNone = 0, kSortPostGather = 1, kSortPostRefine = 2 };
int launch_bucket_sort(Grid &g, const SampleView &sv, int nb_avg, int post, cudaStream_t stream, int *K_out,
                       int shard = 0, int nshards = 1, unsigned long long *n_acc = nullptr);

// lookup_fused.cu: one kernel per lookup batch (search + interpolation in one thread)
void launch_fused(int grid_type, int search, bool sorted, int blocks, int tpb, cudaStream_t stream,
                  const GridView &gv, const SampleView &sv, const SortedView &so, Affine J_grid, double *out,
                  int32_t *out_idx, unsigned long long *stats);

// lookup_staged.cu: XS_SEARCH_S in sorted order (one persistent wave, 256 threads per CTA)
void launch_staged(int grid_type, int blocks, int tpb, cudaStream_t stream, const GridView &gv,
                   const SampleView &sv, const SortedView &so, double *out, int32_t *out_idx,
                   unsigned long long *stats);

// lookup_fused.cu: XSBench history order (XS_SORT_HISTORY)
void launch_history(int grid_type, int search, int hl, int blocks, cudaStream_t stream, const GridView &gv,
                    const SampleView &sv, double *out, int32_t *out_idx, unsigned long long *stats);

// lookup_split.cu: k_search (every pair's lower index into the pair buffer; the paper's
// loop, alone, at full occupancy) then k_interp (gather + interpolate + accumulate)
void launch_search(int grid_type, int search, int blocks, cudaStream_t stream, const GridView &gv,
                   const SortedView &so, const PairView &pv);
void launch_interp(int blocks, cudaStream_t stream, const GridView &gv, const SortedView &so, const PairView &pv,
                   double *out, int32_t *out_idx, unsigned long long *stats);
constexpr int kSearchTpb = 256;
constexpr int kInterpTpb = 256;

// pipeline.cu
// Resident CTAs per SM of kernel f at (tpb threads, smem bytes of dynamic shared memory) on
// the current device; the first call per (device, f, smem) also raises f's dynamic-shared-
// memory limit to smem.  Cached, so a call costs no driver round trip after the first (the
// attribute and occupancy queries used to run on every launch).  A maximum shared-memory
// carveout for every kernel (-DXS_MAX_CARVEOUT) measured 1% slower: the lookup kernel's
// global loads lose L1.
int resident_ctas(const void *f, int tpb, int smem);

// Programmatic dependent launch (PDL) between the kernels of one lookup step: a kernel is
// launched with programmatic stream serialisation, so its CTAs can be scheduled while its
// predecessor drains; every such kernel starts with pdl_wait() (griddepcontrol.wait: blocks
// until the predecessor grid has completed and its memory is visible -- before any read of
// its outputs) and then pdl_trigger() (lets its own successor start launching).  Without
// the launch attribute both are no-ops.  XS_PDL=0 turns it off.
#ifndef XS_PDL
#define XS_PDL 1
#endif
__device__ __forceinline__ void pdl_wait()
{
#if XS_PDL
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
}
__device__ __forceinline__ void pdl_trigger()
{
#if XS_PDL
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
}
template <typename... KArgs, typename... Args>
inline void launch_pdl(void (*kernel)(KArgs...), int grid, int block, int smem, cudaStream_t stream, Args... args)
{
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = XS_PDL ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    XS_CUDA_TRY(cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...));
}
int sm_count_cached();

void run_lookups(Grid &g, int64_t first, int64_t count, uint64_t seed, const xs_opts &o, double *out_macro,
                 int32_t *out_idx, xs_stats *st);
void run_bezier_surface(int ni, int nj, int64_t res_i, int64_t res_j, int dtype, int variant, const void *P,
                        void *out, cudaStream_t s);
void run_bezier_blend(int64_t count, const int32_t *k, const int32_t *n, const void *mu, int dtype, int variant,
                      void *out, cudaStream_t s);
void run_sample(Grid &g, int64_t first, int64_t count, uint64_t seed, double *q, int32_t *mat, cudaStream_t s);
void run_search_points(Grid &g, int64_t count, const double *q, const int32_t *nuc, int search, int32_t *out,
                       cudaStream_t s);

} // namespace xs
