/*
 * xs.h -- C ABI of libxs.so, the B200-native (sm_100a) XSBench-style macroscopic
 * cross-section lookup: the motivating kernel of "Enhancing Performance through
 * Control-Flow Unmerging and Loop Unrolling on GPUs" (CGO 2024).
 *
 * What one lookup computes (DESIGN.md §1 / SURVEY.md §8a, §8c):
 *   1. sample:  s = skip(seed, 2i)  (Listing 7 loop);
 *               q = next LCG draw, mat = pick_mat(next draw)            [XSB]
 *   2. for each nuclide j of material mat (ascending j):
 *        L   = lower index of q in the nuclide's energy grid -- found with the
 *              Listing-1 binary search in one of the
 *              variants below, through the nuclide, unionized or hash grid;
 *        f   = (E[L+1]-q)/(E[L+1]-E[L]);  micro_c = fma(-f, X_c[L+1]-X_c[L], X_c[L+1])
 *        acc_c = fma(micro_c, conc_j, acc_c)
 *   3. v = 1 + first argmax_c acc_c ; hash += v ; pairs += num_nucs[mat]
 * Results are a pure function of (grid seed, lookup seed, i): independent of how a
 * range is split, of the sort mode, the search variant and the number of GPUs.
 *
 * Conventions for every entry point:
 *   - Status: XS_OK (0) or a negative XS_E* code; the message of the last failing
 *     call on this host thread is xs_last_error().  No C++ exception crosses the ABI.
 *   - Devices: a grid belongs to the CUDA device that was current at
 *     xs_grid_create; every call on it switches to that device for its duration.
 *   - Streams: work is enqueued on opts->stream (a cudaStream_t; NULL = the legacy
 *     default stream).  Calls are synchronous: they return after the stream has
 *     drained their work.  A grid owns scratch buffers, so calls on ONE grid must
 *     be serialised by the caller; different grids are independent.
 *   - Memory: the grid owns all of its device memory.  The caller owns every out_*
 *     buffer; "device" buffers must be device (or managed) memory, "any" buffers
 *     may be device, pinned host or pageable host memory.
 */
#ifndef XS_H
#define XS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct xs_grid xs_grid; /* opaque */

/* Grid types, XSBench numbering [XSB]. */
enum { XS_UNIONIZED = 0, XS_NUCLIDE = 1, XS_HASH = 2 };

/* Status codes. */
enum { XS_OK = 0, XS_EINVAL = -1, XS_ENOMEM = -2, XS_ECUDA = -3, XS_EDUP = -4 };

/* Binary-search variants.  All visit the probe sequence of Listing 3 and return the
 * same index (SURVEY.md §8c proof 1); only their control flow differs -- the A/B
 * the paper measures (Listings 4 and 5).                       */
enum {
    XS_SEARCH_M = 0,  /* merged: Listing 3 as written (select-based, Listing 4 shape)  */
    XS_SEARCH_U1 = 1, /* unmerged: each branch its own length update + loop test    */
    XS_SEARCH_U2 = 2, /* unmerged + unrolled x2, 4 paths with own back edges (L. 5) */
    XS_SEARCH_U4 = 3, /* unmerged + unrolled x4 (2^4 leaf paths)        */
    XS_SEARCH_U8 = 4, /* unmerged + unrolled x8 (2^8 leaf paths)                      */
    XS_SEARCH_B = 5,  /* branchless select form of the unmerged update               */
    XS_SEARCH_M2 = 6, /* unroll-only x2 of M (Fig. 7 "unroll" configuration)        */
    XS_SEARCH_M4 = 7, /* unroll-only x4                                             */
    XS_SEARCH_M8 = 8, /* unroll-only x8                                             */
    XS_SEARCH_W = 9,  /* warp-cooperative: in sorted modes a warp
                         whose 32 lookups share a material finds L(q_min) and L(q_max) with
                         two half-warp 17-ary searches over a per-nuclide separator tree
                         (one 128 B node per level), then each lane runs Listing 1 inside
                         [L(q_min), L(q_max)+1].  Nuclide grid only; elsewhere (unsorted,
                         mixed-material warps, unionized/hash grids) it is U2.          */
    XS_SEARCH_H = 10, /* bin-bounded: per nuclide a table Tb[b] = L(b / 2^k), b = 0..2^k,
                         2^k >= n_gridpoints (built at grid creation); q*2^k is exact, so
                         L(q) lies in [Tb[b], Tb[b+1]] for b = floor(q*2^k) and Listing 1
                         (U2) runs on that window -- usually 1-2 points.  XSBench's hash-
                         grid idea (R7) at power-of-two resolution.  On the unionized grid
                         the same table over U bounds the one U search per lookup; on the
                         hash grid (whose 10,000-bin table is the configuration) it is U2. */
    XS_SEARCH_S = 11, /* staged warp window (sorted modes): a warp whose
                         lookups share a material takes q_min, q_max over its lanes; lane t
                         finds [L(q_min), L(q_max)] of nuclide t (H bounds) and copies that
                         window's point records into shared memory, 32 nuclides at a time;
                         each lane then runs Listing 1 (U1) on the staged window energies
                         and interpolates from shared memory.  L(q) is exact because L is
                         monotone in q.  Windows that do not fit, mixed-material warps and
                         unsorted lookups take the H path.                               */
    XS_SEARCH_COUNT = 12
};

/* Lookup ordering (a pure reordering: results are invariant). */
enum {
    XS_SORT_NONE = 0,            /* one thread per lookup in index order (XSBench baseline)  */
    XS_SORT_MATERIAL = 1,        /* bucket by material                                       */
    XS_SORT_MATERIAL_ENERGY = 2, /* bucket by (material, energy bucket): coherent warps      */
    XS_SORT_HISTORY = 3          /* XSBench history order: one thread
                                    per particle running opts.history_len consecutive lookups,
                                    its stream continuing from one lookup to the next (lookup
                                    i of the range = particle i / len, step i % len)        */
};

/* Flags. */
enum {
    XS_FLAG_TIMING = 1, /* fill the per-phase *_ms fields of xs_stats (CUDA events)          */
    XS_FLAG_SPLIT = 2,  /* sorted modes: the split k_search -> k_interp pair instead of the one
                           fused search+interpolation kernel (A/B of the two designs)          */
    XS_FLAG_COARSE = 4  /* XS_SORT_MATERIAL_ENERGY, fused kernel: stop at the coarse bucket
                           order (no k_bucket_refine pass; the lookup kernel then gathers each
                           slot's energy by lookup offset).  A/B of the refine pass; results are
                           identical either way (any order is a valid ordering)               */
};

typedef struct xs_opts {
    int32_t search;      /* XS_SEARCH_*                                                 */
    int32_t sort;        /* XS_SORT_*                                                   */
    void *stream;        /* cudaStream_t, NULL = legacy default stream                  */
    int32_t block;       /* threads per CTA of the lookup kernel: 0 = default (256)     */
    int32_t energy_bins; /* XS_SORT_MATERIAL_ENERGY: energy buckets per material on average,
                            power of two in [1, 4096]; 0 = default (4096).  The 12 x
                            energy_bins buckets are shared out in proportion to each
                            material's expected (lookup, nuclide) pairs                 */
    uint32_t flags;      /* XS_FLAG_*                                                   */
    int32_t history_len; /* XS_SORT_HISTORY: lookups per particle; 0 = default (34)     */
    int32_t shard_index; /* key-range sharding (XS_SORT_MATERIAL_ENERGY + XS_SEARCH_S, the
                            refined order; a strong-scaling split of one lookup range over
                            shard_count processes): the call draws EVERY lookup
                            of [first, first + count) but orders and looks up only those whose
                            (material, energy) bucket lies in the shard_index-th of
                            shard_count equal bucket ranges -- each shard then holds ~count /
                            shard_count lookups at the full range's energy density.  stats
                            cover the shard's lookups (stats.lookups = how many); rows of
                            out_macro_xs (device memory only; out_idx unsupported) of the
                            other lookups are left untouched.
                            The shards' hashes, pairs and lookups sum to the unsharded call's.
                            0 <= shard_index < shard_count                              */
    int32_t shard_count; /* 0 or 1 = no sharding (the default)                          */
} xs_opts;

typedef struct xs_stats {
    uint64_t hash;    /* sum over the range of v = 1 + argmax (integer, order-free)          */
    uint64_t lookups; /* number of lookups processed (= count)                              */
    uint64_t pairs;   /* sum of num_nucs[mat] = (lookup, nuclide) pairs interpolated         */
    double device_ms; /* CUDA-event time of the whole call on opts->stream                   */
    double sample_ms; /* XS_FLAG_TIMING: sampling + ordering kernels                          */
    double lookup_ms; /* XS_FLAG_TIMING: the lookup kernel(s): k_lookup, or k_search + k_interp */
    double search_ms; /* XS_FLAG_TIMING: k_search alone (XS_FLAG_SPLIT; else 0)              */
    double copy_ms;   /* XS_FLAG_TIMING: device->host copy of out_macro_xs (host outputs)      */
    int32_t launches; /* CUDA kernels this call launched (all kinds)                          */
    int32_t reserved;
} xs_stats;

typedef struct xs_grid_info {
    int64_t n_nuclides;
    int64_t n_gridpoints;
    int64_t n_points;        /* n_nuclides * n_gridpoints                 */
    int64_t hash_bins;
    uint64_t seed;
    uint64_t device_bytes;   /* device memory owned by the grid (no scratch) */
    int32_t grid_type;
    int32_t device;
    int32_t max_num_nucs;    /* 34 (small tables) or 321 (large tables)    */
    int32_t num_nucs[12];
} xs_grid_info;

/* Fill *opts with the defaults: XS_SEARCH_S, XS_SORT_MATERIAL_ENERGY, legacy stream, no flags. */
void xs_opts_default(xs_opts *opts);

/* Build a grid on the current CUDA device:
 *   point p = (i, k) takes the draws at grid-stream positions 6p .. 6p+5 (energy, then
 *   total, elastic, absorption, fission, nu-fission); each nuclide is sorted by energy;
 *   concentrations continue the stream at 6N.  grid_type adds the unionized energy-
 *   index table (U[N], IDX[N][n_nuclides]) or the hash table (H[10000][n_nuclides]).
 * Valid: n_nuclides == 68 (small tables) or >= 355 (large tables); n_gridpoints >= 2;
 *        n_nuclides * n_gridpoints < 2^31; grid_type in {0,1,2}.
 * Returns NULL on error (xs_last_error(): XS_EINVAL / XS_ENOMEM / XS_ECUDA / XS_EDUP
 * -- a duplicated energy within one nuclide, probability ~ n^2/2^64).  Setup is not
 * part of the timed hot path (XSBench grid_init_do_not_profile [XSB]). */
xs_grid *xs_grid_create(int64_t n_nuclides, int64_t n_gridpoints, int grid_type, uint64_t seed);

/* As xs_grid_create with an explicit hash-bin count (>= 1; XS_HASH only). */
xs_grid *xs_grid_create_ex(int64_t n_nuclides, int64_t n_gridpoints, int grid_type,
                           uint64_t seed, int64_t hash_bins);

/* NULL-safe; frees every device buffer of the grid. */
void xs_grid_destroy(xs_grid *grid);

/* Message of the last non-OK call on this host thread ("" if none). */
const char *xs_last_error(void);

/* Lookups 0 .. n_lookups-1 with default options on the legacy stream.
 * out_macro_xs: any memory, [n_lookups][5] row-major fp64, or NULL.
 * out_hash: host, required; receives sum of v over the batch.
 * n_lookups >= 0 (0 gives hash 0). */
int xs_lookup_batch(const xs_grid *grid, int64_t n_lookups, uint64_t seed,
                    double *out_macro_xs, uint64_t *out_hash);

/* Lookups first .. first+count-1 (0 <= first, 0 <= count, first+count <= 2^62).
 * opts: NULL = defaults.  out_macro_xs: any memory, [count][5] indexed by i - first,
 * or NULL.  out_stats: host, may be NULL. */
int xs_lookup_range(const xs_grid *grid, int64_t first, int64_t count, uint64_t seed,
                    const xs_opts *opts, double *out_macro_xs, xs_stats *out_stats);

/* Debug/parity: the lower index L found for every (lookup, nuclide) pair.
 * out_idx: device, [count][max_num_nucs] int32 indexed by i - first; entry j is the
 * index for mats[mat][j]; entries j >= num_nucs[mat] are -1. */
int xs_lookup_indices(const xs_grid *grid, int64_t first, int64_t count, uint64_t seed,
                      const xs_opts *opts, int32_t *out_idx);

/* Debug/parity: the sampled energy and material of lookups first .. first+count-1.
 * out_q: device fp64 [count]; out_mat: device int32 [count]. */
int xs_sample(const xs_grid *grid, int64_t first, int64_t count, uint64_t seed,
              double *out_q, int32_t *out_mat, void *stream);

/* Debug/parity: lower index of nuclide nuc[t] at an arbitrary energy q[t] (any fp64,
 * including values outside [0,1]) through the grid's own path (nuclide search,
 * unionized table or hash window) and search variant `search`.
 * q, nuc, out_L: device arrays of length count. */
int xs_search_points(const xs_grid *grid, int64_t count, const double *q, const int32_t *nuc,
                     int32_t search, int32_t *out_L, void *stream);

/* Position-weighted 64-bit checksum of every table the grid holds (multi-GPU
 * replica check: all ranks must agree). */
int xs_grid_checksum(const xs_grid *grid, uint64_t *out);

int xs_grid_get_info(const xs_grid *grid, xs_grid_info *out);

/* Debug/parity: copy the grid to host arrays (each may be NULL).
 * E [n_nuclides][n_gridpoints], X [n_nuclides][n_gridpoints][5],
 * mats [12][max_num_nucs] (-1 padded), concs [12][max_num_nucs] (0 padded). */
int xs_grid_export(const xs_grid *grid, double *E, double *X, int32_t *mats, double *concs);

/* Debug/parity: U [n_points] + IDX [n_points][n_nuclides] (XS_UNIONIZED) or
 * H [hash_bins][n_nuclides] (XS_HASH); host arrays, each may be NULL. */
int xs_grid_export_aux(const xs_grid *grid, double *U, int32_t *IDX, int32_t *H);

/* ---------------------------------------------------------------------------------
 * The paper's second u&u example: the bezier-surface loop (Listing 2, PAPER.md:160-185;
 * SURVEY.md §8f NEXT 4; DESIGN.md §6.9 and readings BZ1-BZ5).  Off the north star: a
 * synthetic A/B of the loop transformation.  BezierBlend(k, mu, n) = Listing 2 (from
 * blend = 1, nn = n, kn = k, nkn = n - k) * mu^k * (1 - mu)^(n - k), powers by repeated
 * multiplication; surface(i, j)[c] = sum_ki sum_kj (P[ki][kj][c] * B(ki, mu_i, ni)) *
 * B(kj, mu_j, nj), ki-major, mu_i = i / (res_i - 1).  Every variant performs the same
 * floating-point operations in the same order: results are bit-identical across variants
 * and to the CPU oracle.
 * --------------------------------------------------------------------------------- */
enum {
    XS_BZ_M = 0,  /* Listing 2 as written                                              */
    XS_BZ_M2 = 1, /* unroll-only x2                                                    */
    XS_BZ_U1 = 2, /* unmerge-only                                                      */
    XS_BZ_U2 = 3, /* u&u x2: the unrolled copy specialised per path (Figure 5)         */
    XS_BZ_S = 4,  /* one loop per condition state (the u -> infinity limit)            */
    XS_BZ_T = 5,  /* B200 design: per-tile blends in shared memory, then contraction   */
    XS_BZ_COUNT = 6
};
enum { XS_F64 = 0, XS_F32 = 1 }; /* element type of the bezier buffers */

/* Evaluate a res_i x res_j bezier surface.
 *   ni, nj   in [0, 32]: the control net has (ni+1) x (nj+1) points
 *   res_i, res_j >= 2, res_i * res_j < 2^40
 *   ctrl     device, [(ni+1)][(nj+1)][3] of dtype (row-major)
 *   out      device, [res_i][res_j][3] of dtype (written in full)
 *   dtype    XS_F64 or XS_F32 (every operation rounded in that type, no contraction)
 *   variant  XS_BZ_*
 * Enqueued on `stream` and synchronised before returning.  XS_EINVAL on a bad argument. */
int xs_bezier_surface(int32_t ni, int32_t nj, int64_t res_i, int64_t res_j, int32_t dtype, int32_t variant,
                      const void *ctrl, void *out, void *stream);

/* Loop-level parity: out[t] = BezierBlend(k[t], mu[t], n[t]), or the bare Listing-2
 * loop value when mu is NULL.  k, n, mu, out: device arrays of length count (mu and out
 * of dtype).  The loop runs n[t] trips: callers keep 0 <= k[t] and n[t] <= 2^20
 * (device contents are not inspected).  XS_BZ_T evaluates the loop as XS_BZ_M. */
int xs_bezier_blend(int64_t count, const int32_t *k, const int32_t *n, const void *mu, int32_t dtype,
                    int32_t variant, void *out, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* XS_H */
