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
    double *U = nullptr;
    int32_t *IDX = nullptr;
    int32_t *H = nullptr;
    int32_t *mats = nullptr;
    double *concs = nullptr;
    int32_t *num_nucs_d = nullptr;

    // per-grid scratch (grown on demand; calls on one grid are serialised by the caller)
    uint64_t *stats_d = nullptr;     // [4] hash, pairs
    uint64_t *stats_h = nullptr;     // pinned mirror
    double *sq = nullptr;            // sorted energies       [cap]
    uint32_t *si = nullptr;          // sorted lookup offsets [cap]
    uint32_t *hist = nullptr;        // per-CTA bucket histograms [ctas][K]
    uint32_t *base = nullptr;        // [K + 16]: bucket bases, then material bases
    int64_t cap = 0, hist_cap = 0;
    double *stage = nullptr;         // device staging for host outputs
    int64_t stage_cap = 0;
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
struct GridView {
    const double *__restrict__ E;
    const double *__restrict__ pts;
    const double *__restrict__ U;
    const int32_t *__restrict__ IDX;
    const int32_t *__restrict__ H;
    const int32_t *__restrict__ mats;
    const double *__restrict__ concs;
    const int32_t *__restrict__ num_nucs;
    int32_t n;        // gridpoints per nuclide
    int32_t n_nuc;
    int32_t N;        // n_nuc * n
    int32_t bins;
    int32_t max_nucs;
    int32_t pad_;
    double du;        // 1.0 / bins
};

struct SampleView {
    uint64_t seed;
    int64_t first;
    int64_t count;
    double T[kMaterials]; // pick_mat thresholds, T[0] unused
};

GridView make_view(const Grid &g);
SampleView make_sample_view(const Grid &g, uint64_t seed, int64_t first, int64_t count);

// grid.cu
void build_grid(Grid &g);
void free_grid(Grid &g);
uint64_t grid_checksum(const Grid &g);

// lookup.cu
void run_lookups(Grid &g, int64_t first, int64_t count, uint64_t seed, const xs_opts &o, double *out_macro,
                 int32_t *out_idx, xs_stats *st);
void run_sample(Grid &g, int64_t first, int64_t count, uint64_t seed, double *q, int32_t *mat, cudaStream_t s);
void run_search_points(Grid &g, int64_t count, const double *q, const int32_t *nuc, int search, int32_t *out,
                       cudaStream_t s);

} // namespace xs
