// api.cu -- the extern "C" boundary declared in include/xs.h.
//
// Argument validation, device/stream plumbing and error translation only; every step
// of the lookup path runs in the kernels of grid.cu and lookup.cu.
#include <stdio.h>

#include <new>
#include <string>

#include "xs_internal.cuh"

struct xs_grid {
    xs::Grid g;
};

namespace xs {

static thread_local std::string t_err;
static thread_local int t_code = 0;

void set_error(int code, const std::string &msg)
{
    t_code = code;
    t_err = msg;
}
void clear_error()
{
    t_code = 0;
    t_err.clear();
}

template <class F> static int guarded(F &&f)
{
    try {
        clear_error();
        f();
        return XS_OK;
    } catch (const Error &e) {
        set_error(e.code, e.msg);
        return e.code;
    } catch (const std::bad_alloc &) {
        set_error(XS_ENOMEM, "host allocation failed");
        return XS_ENOMEM;
    } catch (...) {
        set_error(XS_ECUDA, "unknown failure");
        return XS_ECUDA;
    }
}

static void check_grid(const xs_grid *grid) { XS_CHECK_ARG(grid != nullptr, "grid is NULL"); }

static void check_range(int64_t first, int64_t count)
{
    XS_CHECK_ARG(first >= 0, "first must be >= 0");
    XS_CHECK_ARG(count >= 0, "count must be >= 0");
    XS_CHECK_ARG(first <= (int64_t(1) << 62) - count, "first + count must be <= 2^62");
}

} // namespace xs

using namespace xs;

extern "C" {

void xs_opts_default(xs_opts *o)
{
    if (!o)
        return;
    o->search = XS_SEARCH_S;
    o->sort = XS_SORT_MATERIAL_ENERGY;
    o->stream = nullptr;
    o->block = 0;
    o->energy_bins = 0;
    o->flags = 0;
    o->history_len = 0;
    o->shard_index = 0;
    o->shard_count = 1;
}

const char *xs_last_error(void) { return t_err.c_str(); }

xs_grid *xs_grid_create_ex(int64_t n_nuclides, int64_t n_gridpoints, int grid_type, uint64_t seed, int64_t hash_bins)
{
    xs_grid *out = nullptr;
    int rc = guarded([&] {
        XS_CHECK_ARG(n_nuclides == 68 || n_nuclides >= 355,
                     "n_nuclides must be 68 (small tables) or >= 355 (large tables)");
        XS_CHECK_ARG(n_gridpoints >= 2, "n_gridpoints must be >= 2");
        XS_CHECK_ARG(n_nuclides * n_gridpoints < (int64_t(1) << 31), "n_nuclides * n_gridpoints must be < 2^31");
        XS_CHECK_ARG(grid_type == XS_UNIONIZED || grid_type == XS_NUCLIDE || grid_type == XS_HASH,
                     "grid_type must be 0 (unionized), 1 (nuclide) or 2 (hash)");
        XS_CHECK_ARG(hash_bins >= 1 && hash_bins < (int64_t(1) << 24), "hash_bins must be in [1, 2^24)");
        XS_CHECK_ARG(grid_type != XS_UNIONIZED || n_nuclides * n_gridpoints * n_nuclides < (int64_t(1) << 40),
                     "unionized index table too large");
        int ndev = 0;
        cudaError_t e = cudaGetDeviceCount(&ndev);
        if (e != cudaSuccess || ndev == 0) {
            cudaGetLastError();
            throw Error{XS_ECUDA, std::string("no CUDA device: ") + cudaGetErrorString(e)};
        }
        xs_grid *gr = new xs_grid();
        Grid &g = gr->g;
        XS_CUDA_TRY(cudaGetDevice(&g.device));
        g.n_nuc = n_nuclides;
        g.n = n_gridpoints;
        g.N = n_nuclides * n_gridpoints;
        g.grid_type = grid_type;
        g.seed = seed;
        g.bins = hash_bins;
        try {
            build_grid(g);
        } catch (...) {
            free_grid(g);
            delete gr;
            throw;
        }
        out = gr;
    });
    return rc == XS_OK ? out : nullptr;
}

xs_grid *xs_grid_create(int64_t n_nuclides, int64_t n_gridpoints, int grid_type, uint64_t seed)
{
    return xs_grid_create_ex(n_nuclides, n_gridpoints, grid_type, seed, 10000);
}

void xs_grid_destroy(xs_grid *grid)
{
    if (!grid)
        return;
    DeviceGuard dg(grid->g.device);
    free_grid(grid->g);
    delete grid;
}

int xs_lookup_range(const xs_grid *grid, int64_t first, int64_t count, uint64_t seed, const xs_opts *opts,
                    double *out_macro_xs, xs_stats *out_stats)
{
    return guarded([&] {
        check_grid(grid);
        check_range(first, count);
        xs_opts o;
        xs_opts_default(&o);
        if (opts)
            o = *opts;
        DeviceGuard dg(grid->g.device);
        run_lookups(const_cast<Grid &>(grid->g), first, count, seed, o, out_macro_xs, nullptr, out_stats);
    });
}

int xs_lookup_batch(const xs_grid *grid, int64_t n_lookups, uint64_t seed, double *out_macro_xs, uint64_t *out_hash)
{
    return guarded([&] {
        XS_CHECK_ARG(out_hash != nullptr, "out_hash is required");
        xs_stats st{};
        int rc = xs_lookup_range(grid, 0, n_lookups, seed, nullptr, out_macro_xs, &st);
        if (rc != XS_OK)
            throw Error{rc, t_err};
        *out_hash = st.hash;
    });
}

int xs_lookup_indices(const xs_grid *grid, int64_t first, int64_t count, uint64_t seed, const xs_opts *opts,
                      int32_t *out_idx)
{
    return guarded([&] {
        check_grid(grid);
        check_range(first, count);
        XS_CHECK_ARG(out_idx != nullptr || count == 0, "out_idx is required");
        xs_opts o;
        xs_opts_default(&o);
        if (opts)
            o = *opts;
        DeviceGuard dg(grid->g.device);
        run_lookups(const_cast<Grid &>(grid->g), first, count, seed, o, nullptr, out_idx, nullptr);
    });
}

int xs_sample(const xs_grid *grid, int64_t first, int64_t count, uint64_t seed, double *out_q, int32_t *out_mat,
              void *stream)
{
    return guarded([&] {
        check_grid(grid);
        check_range(first, count);
        XS_CHECK_ARG((out_q && out_mat) || count == 0, "out_q and out_mat are required");
        DeviceGuard dg(grid->g.device);
        run_sample(const_cast<Grid &>(grid->g), first, count, seed, out_q, out_mat, (cudaStream_t)stream);
    });
}

int xs_search_points(const xs_grid *grid, int64_t count, const double *q, const int32_t *nuc, int32_t search,
                     int32_t *out_L, void *stream)
{
    return guarded([&] {
        check_grid(grid);
        XS_CHECK_ARG(count >= 0, "count must be >= 0");
        XS_CHECK_ARG((q && nuc && out_L) || count == 0, "q, nuc and out_L are required");
        DeviceGuard dg(grid->g.device);
        run_search_points(const_cast<Grid &>(grid->g), count, q, nuc, search, out_L, (cudaStream_t)stream);
    });
}

int xs_grid_checksum(const xs_grid *grid, uint64_t *out)
{
    return guarded([&] {
        check_grid(grid);
        XS_CHECK_ARG(out != nullptr, "out is required");
        DeviceGuard dg(grid->g.device);
        *out = grid_checksum(grid->g);
    });
}

int xs_grid_get_info(const xs_grid *grid, xs_grid_info *out)
{
    return guarded([&] {
        check_grid(grid);
        XS_CHECK_ARG(out != nullptr, "out is required");
        const Grid &g = grid->g;
        out->n_nuclides = g.n_nuc;
        out->n_gridpoints = g.n;
        out->n_points = g.N;
        out->hash_bins = g.bins;
        out->seed = g.seed;
        out->device_bytes = g.device_bytes;
        out->grid_type = g.grid_type;
        out->device = g.device;
        out->max_num_nucs = g.max_nucs;
        for (int m = 0; m < 12; m++)
            out->num_nucs[m] = g.num_nucs[m];
    });
}

int xs_grid_export(const xs_grid *grid, double *E, double *X, int32_t *mats, double *concs)
{
    return guarded([&] {
        check_grid(grid);
        const Grid &g = grid->g;
        DeviceGuard dg(g.device);
        if (E)
            XS_CUDA_TRY(cudaMemcpy(E, g.E, (size_t)g.N * 8, cudaMemcpyDeviceToHost));
        if (X)
            // pts records are {E, x0..x4}: copy the 5 channels of every 48 B record
            XS_CUDA_TRY(cudaMemcpy2D(X, 5 * sizeof(double), g.pts + 1, 6 * sizeof(double), 5 * sizeof(double),
                                     (size_t)g.N, cudaMemcpyDeviceToHost));
        if (mats)
            XS_CUDA_TRY(cudaMemcpy(mats, g.mats, (size_t)12 * g.max_nucs * 4, cudaMemcpyDeviceToHost));
        if (concs)
            XS_CUDA_TRY(cudaMemcpy(concs, g.concs, (size_t)12 * g.max_nucs * 8, cudaMemcpyDeviceToHost));
    });
}

int xs_grid_export_aux(const xs_grid *grid, double *U, int32_t *IDX, int32_t *H)
{
    return guarded([&] {
        check_grid(grid);
        const Grid &g = grid->g;
        DeviceGuard dg(g.device);
        if (U) {
            XS_CHECK_ARG(g.U != nullptr, "grid has no unionized table");
            XS_CUDA_TRY(cudaMemcpy(U, g.U, (size_t)g.N * 8, cudaMemcpyDeviceToHost));
        }
        if (IDX) {
            XS_CHECK_ARG(g.IDX != nullptr, "grid has no unionized index table");
            XS_CUDA_TRY(cudaMemcpy(IDX, g.IDX, (size_t)g.N * g.n_nuc * 4, cudaMemcpyDeviceToHost));
        }
        if (H) {
            XS_CHECK_ARG(g.H != nullptr, "grid has no hash table");
            XS_CUDA_TRY(cudaMemcpy(H, g.H, (size_t)g.bins * g.n_nuc * 4, cudaMemcpyDeviceToHost));
        }
    });
}

int xs_bezier_surface(int32_t ni, int32_t nj, int64_t res_i, int64_t res_j, int32_t dtype, int32_t variant,
                      const void *ctrl, void *out, void *stream)
{
    return guarded([&] {
        XS_CHECK_ARG(ni >= 0 && ni <= 32 && nj >= 0 && nj <= 32, "ni and nj must be in [0, 32]");
        XS_CHECK_ARG(res_i >= 2 && res_j >= 2, "res_i and res_j must be >= 2");
        XS_CHECK_ARG(res_i < (int64_t(1) << 40) / res_j, "res_i * res_j must be < 2^40");
        XS_CHECK_ARG(dtype == XS_F64 || dtype == XS_F32, "dtype must be XS_F64 or XS_F32");
        XS_CHECK_ARG(variant >= 0 && variant < XS_BZ_COUNT, "unknown bezier variant");
        XS_CHECK_ARG(ctrl != nullptr && out != nullptr, "ctrl and out are required");
        const cudaStream_t s = (cudaStream_t)stream;
        run_bezier_surface(ni, nj, res_i, res_j, dtype, variant, ctrl, out, s);
        XS_CUDA_TRY(cudaStreamSynchronize(s));
    });
}

int xs_bezier_blend(int64_t count, const int32_t *k, const int32_t *n, const void *mu, int32_t dtype,
                    int32_t variant, void *out, void *stream)
{
    return guarded([&] {
        XS_CHECK_ARG(count >= 0, "count must be >= 0");
        XS_CHECK_ARG((k && n && out) || count == 0, "k, n and out are required");
        XS_CHECK_ARG(dtype == XS_F64 || dtype == XS_F32, "dtype must be XS_F64 or XS_F32");
        XS_CHECK_ARG(variant >= 0 && variant < XS_BZ_COUNT, "unknown bezier variant");
        const cudaStream_t s = (cudaStream_t)stream;
        run_bezier_blend(count, k, n, mu, dtype, variant, out, s);
        XS_CUDA_TRY(cudaStreamSynchronize(s));
    });
}

} // extern "C"
