// pipeline.cu -- host orchestration of one xs_lookup_range call.
//
//   XS_SORT_NONE                   k_lookup<unsorted>  (sampling fused in)
//   XS_SORT_MATERIAL[_ENERGY]      bucket sort (4 kernels, + k_bucket_refine)  ->  k_lookup<sorted>
//     + XS_FLAG_SPLIT              bucket sort + gather     ->  k_search -> k_interp
// A range is processed in chunks (slot indices are uint32; scratch stays bounded).  The
// fused path reads the material bases from device memory (no host round trip); the split
// path brings them back (52 B) to size the pair buffer exactly.
#include <algorithm>
#include <cstdlib>
#include <mutex>
#include <vector>

#include "lookup_common.cuh"

namespace xs {

// ---- debug kernels -------------------------------------------------------------------------
__global__ void k_sample(SampleView sv, double *__restrict__ q_out, int32_t *__restrict__ mat_out)
{
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < sv.count;
         j += (int64_t)gridDim.x * blockDim.x) {
        double q;
        int mat;
        sample_lookup(lookup_state(sv, j), sv, q, mat);
        q_out[j] = q;
        mat_out[j] = mat;
    }
}

template <int GRID, int SEARCH>
__global__ void k_search_points(GridView gv, int64_t count, const double *__restrict__ q,
                                const int32_t *__restrict__ nuc, int32_t *__restrict__ out)
{
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < count; t += (int64_t)gridDim.x * blockDim.x) {
        const double qq = q[t];
        const int nu = nuc[t];
        out[t] = lower_index<GRID, SEARCH>(gv, make_row(gv, nu), qq, union_index<GRID, SEARCH>(gv, qq));
    }
}

using SearchPtsFn = void (*)(GridView, int64_t, const double *, const int32_t *, int32_t *);

template <int GRID> static SearchPtsFn pick_pts(int search)
{
    switch (search) {
    case XS_SEARCH_M: return k_search_points<GRID, XS_SEARCH_M>;
    case XS_SEARCH_U1: return k_search_points<GRID, XS_SEARCH_U1>;
    case XS_SEARCH_U2: return k_search_points<GRID, XS_SEARCH_U2>;
    case XS_SEARCH_U4: return k_search_points<GRID, XS_SEARCH_U4>;
    case XS_SEARCH_U8: return k_search_points<GRID, XS_SEARCH_U8>;
    case XS_SEARCH_B: return k_search_points<GRID, XS_SEARCH_B>;
    case XS_SEARCH_M2: return k_search_points<GRID, XS_SEARCH_M2>;
    case XS_SEARCH_M4: return k_search_points<GRID, XS_SEARCH_M4>;
    case XS_SEARCH_M8: return k_search_points<GRID, XS_SEARCH_M8>;
    case XS_SEARCH_W: return k_search_points<GRID, XS_SEARCH_W>;
    default: return k_search_points<GRID, XS_SEARCH_H>;
    }
}

// ---- helpers ---------------------------------------------------------------------------------
int sm_count_cached()
{
    static int cache[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    int &c = cache[dev & 63];
    if (!c) {
        int sms = 0;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        c = sms > 0 ? sms : 148;
    }
    return c;
}

static int sm_count() { return sm_count_cached(); }

int resident_ctas(const void *f, int tpb, int smem)
{
    struct Entry {
        const void *f;
        int dev, tpb, smem, per_sm;
    };
    static std::mutex mu;
    static std::vector<Entry> cache;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    for (const Entry &e : cache)
        if (e.f == f && e.dev == dev && e.tpb == tpb && e.smem == smem)
            return e.per_sm;
    XS_CUDA_TRY(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
#ifdef XS_MAX_CARVEOUT
    XS_CUDA_TRY(cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, cudaSharedmemCarveoutMaxShared));
#endif
    int per_sm = 0;
    XS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, tpb, smem));
    per_sm = std::max(per_sm, 1);
    cache.push_back(Entry{f, dev, tpb, smem, per_sm});
    return per_sm;
}

static bool is_device_accessible(const void *p)
{
    cudaPointerAttributes a{};
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

static int log2_exact(int v)
{
    int l = 0;
    while ((1 << l) < v)
        l++;
    return ((1 << l) == v) ? l : -1;
}

static int blocks_for(int64_t work, int tpb, int per_sm)
{
    const int64_t want = (work + tpb - 1) / tpb;
    return (int)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)sm_count() * per_sm));
}

template <class T> static void grow(T *&p, int64_t &cap, int64_t need)
{
    if (cap >= need)
        return;
    cudaFree(p);
    p = nullptr;
    cap = 0;
    XS_CUDA_TRY(cudaMalloc(&p, (size_t)need * sizeof(T)));
    cap = need;
}

constexpr int64_t kChunkFused = int64_t(1) << 28;  // uint32 slots
// one sort per 2^28 lookups: a 2^25 cap kept the 4 B slot array L2-sized and halved the
// sort time of 100M lookups, but the coarser ordering cost more in the lookup kernel
constexpr int64_t kChunkSorted = int64_t(1) << 28;
constexpr int64_t kChunkSplit = int64_t(1) << 25;  // pair buffer <= 33.5M x 321 x 4 B
constexpr int64_t kChunkHost = int64_t(1) << 22;   // staging for host outputs (x2 buffers)

static void run_lookups_impl(Grid &g, int64_t first, int64_t count, uint64_t seed, const xs_opts &o,
                             double *out_macro, int32_t *out_idx, xs_stats *st)
{
    XS_CHECK_ARG(o.search >= 0 && o.search < XS_SEARCH_COUNT, "opts.search out of range");
    XS_CHECK_ARG(o.sort >= XS_SORT_NONE && o.sort <= XS_SORT_HISTORY, "opts.sort out of range");
    const bool history = o.sort == XS_SORT_HISTORY;
    const int hl = o.history_len ? o.history_len : 34;
    XS_CHECK_ARG(!history || (hl >= 1 && hl <= (1 << 20)), "opts.history_len must be in [1, 2^20]");
    // key-range sharding (xs.h): the refined (material, energy) order with the staged kernel
    const int nshards = o.shard_count > 1 ? o.shard_count : 1;
    const int shard = nshards > 1 ? o.shard_index : 0;
    const bool sharded = nshards > 1;
    XS_CHECK_ARG(o.shard_count >= 0 && o.shard_index >= 0 && (o.shard_count <= 1 ? o.shard_index == 0 : shard < nshards),
                 "opts.shard_index must be in [0, shard_count)");
    XS_CHECK_ARG(!sharded || (o.sort == XS_SORT_MATERIAL_ENERGY && o.search == XS_SEARCH_S && o.energy_bins != 1 &&
                              !(o.flags & (XS_FLAG_SPLIT | XS_FLAG_COARSE))),
                 "key-range sharding needs sort = XS_SORT_MATERIAL_ENERGY, search = XS_SEARCH_S, no split / coarse");
    XS_CHECK_ARG(!sharded || out_idx == nullptr, "key-range sharding does not write out_idx");
    const int tpb = o.block ? o.block : 256;
    XS_CHECK_ARG(tpb == 64 || tpb == 128 || tpb == 256, "opts.block must be 64, 128 or 256");
    const int nb = (o.sort == XS_SORT_MATERIAL_ENERGY) ? (o.energy_bins ? o.energy_bins : kMaxEnergyBins) : 1;
    const int nb_log2 = log2_exact(nb);
    XS_CHECK_ARG(nb_log2 >= 0 && nb <= kMaxEnergyBins, "opts.energy_bins must be a power of two <= 4096");
    cudaStream_t stream = (cudaStream_t)o.stream;
    const bool timing = (o.flags & XS_FLAG_TIMING) != 0;
    const bool sorted = o.sort == XS_SORT_MATERIAL || o.sort == XS_SORT_MATERIAL_ENERGY;
    const bool fused = !sorted || !(o.flags & XS_FLAG_SPLIT);
    const bool host_out = out_macro && !is_device_accessible(out_macro);
    XS_CHECK_ARG(!sharded || !host_out, "key-range sharding writes device outputs only");
    int64_t chunk = fused ? (sorted ? kChunkSorted : kChunkFused) : kChunkSplit;
    if (host_out)
        chunk = std::min(chunk, kChunkHost);
    // test hook: XS_TEST_MAX_CHUNK forces small chunks so the chunk-boundary paths (offsets,
    // host-output double buffering, history alignment) are checked at tiny sizes
    if (const char *env = std::getenv("XS_TEST_MAX_CHUNK")) {
        const long long v = std::atoll(env);
        if (v > 0)
            chunk = std::min<int64_t>(chunk, v);
    }
    if (count > chunk) { // equal chunks (no small tail chunk)
        const int64_t nch = (count + chunk - 1) / chunk;
        chunk = (count + nch - 1) / nch;
    }
    if (history && count > chunk) // whole particles per chunk: history stream positions stay global
        chunk = std::max<int64_t>(hl, chunk / hl * hl);
    const GridView gv = make_view(g);
    int launches = 0;
    double sample_ms = 0, lookup_ms = 0, search_ms = 0, copy_ms = 0;

    if (host_out) {
        grow(g.stage, g.stage_cap, std::min(count, chunk) * 5 * 2);
        if (!g.copy_stream) {
            XS_CUDA_TRY(cudaStreamCreateWithFlags(&g.copy_stream, cudaStreamNonBlocking));
            for (int b = 0; b < 2; b++) {
                XS_CUDA_TRY(cudaEventCreateWithFlags(&g.ev_done[b], cudaEventDisableTiming));
                XS_CUDA_TRY(cudaEventCreateWithFlags(&g.ev_copied[b], cudaEventDisableTiming));
            }
        }
    }
    bool copied_pending[2] = {false, false};
    bool published = false; // the last S chunk wrote the stats to the (mapped) pinned mirror
    const int64_t stage_half = std::min(count, chunk) * 5;
    if (!g.mb_h)
        XS_CUDA_TRY(cudaMallocHost(&g.mb_h, 32 * sizeof(uint32_t)));

    XS_CUDA_TRY(cudaEventRecord(g.ev[0], stream));
    XS_CUDA_TRY(cudaMemsetAsync(g.stats_d, 0, 3 * sizeof(uint64_t), stream)); // hash, pairs, shard lookups
    if (out_idx && count > 0)
        XS_CUDA_TRY(cudaMemsetAsync(out_idx, 0xFF, (size_t)count * g.max_nucs * sizeof(int32_t), stream));
    unsigned long long *stats = (unsigned long long *)g.stats_d;

    for (int64_t c0 = 0, ci = 0; c0 < count; c0 += chunk, ci++) {
        const int64_t cn = std::min(chunk, count - c0);
        const SampleView sv = make_sample_view(g, seed, first + c0, cn);
        const int buf = (int)(ci & 1);
        double *stage = g.stage + buf * stage_half;
        if (host_out && copied_pending[buf]) // the copy out of this buffer must be done
            XS_CUDA_TRY(cudaStreamWaitEvent(stream, g.ev_copied[buf], 0));
        double *outp = out_macro ? (host_out ? stage : out_macro + c0 * 5) : nullptr;
        int32_t *idxp = out_idx ? out_idx + c0 * g.max_nucs : nullptr;
        SortedView so{};
        XS_CUDA_TRY(cudaEventRecord(g.ev[1], stream));
        if (sorted) {
            int K = 0;
            const bool refine = fused && o.sort == XS_SORT_MATERIAL_ENERGY && nb > 1 && !(o.flags & XS_FLAG_COARSE);
            launches += launch_bucket_sort(g, sv, nb, !fused ? kSortPostGather : (refine ? kSortPostRefine : kSortPostNone),
                                           stream, &K, shard, nshards, (unsigned long long *)(g.stats_d + 2));
            so.q = (!fused || refine) ? g.qs : nullptr; // q in slot order when the sort wrote it
            so.q_of = refine ? nullptr : g.sq;
            so.slot = g.si;
            so.mb_dev = g.base + K;
            so.work = reinterpret_cast<int *>(g.stats_d + 4); // zeroed by k_bucket_count
            so.count_dev = sharded ? g.base + K + kMaterials : nullptr; // the shard's slots
            if (fused && o.search == XS_SEARCH_S && c0 + chunk >= count) { // the last chunk of S
                so.done = reinterpret_cast<unsigned int *>(g.stats_d + 5);   // publishes the stats
                so.pub = reinterpret_cast<unsigned long long *>(g.stats_h);
                published = true;
            }
            if (!fused) {
                XS_CUDA_TRY(cudaMemcpyAsync(g.mb_h, g.base + K, (kMaterials + 1) * sizeof(uint32_t),
                                            cudaMemcpyDeviceToHost, stream));
                XS_CUDA_TRY(cudaStreamSynchronize(stream));
                for (int m = 0; m <= kMaterials; m++)
                    so.matbase[m] = g.mb_h[m];
            }
        }
        XS_CUDA_TRY(cudaEventRecord(g.ev[2], stream));
        XS_CUDA_TRY(cudaEventRecord(g.ev[3], stream));
        if (history) {
            // chunk boundaries are multiples of hl (chunk >= 2^22 > hl, rounded below), so a
            // particle never straddles two chunks
            const int64_t particles = (cn + hl - 1) / hl;
            launch_history(g.grid_type, o.search, hl, blocks_for(particles, 256, 32), stream, gv, sv, outp, idxp,
                           stats);
            launches += 1;
        } else if (fused) {
            // sorted: a persistent grid (one resident wave) pulling work chunks;
            // unsorted: 4 waves of grid-stride CTAs
            const int blocks = blocks_for(cn, tpb, sorted ? (1024 / tpb) : (2048 / tpb) * 4);
            const Affine Jg = lcg_jump(2 * (uint64_t)blocks * tpb);
            launch_fused(g.grid_type, o.search, sorted, blocks, tpb, stream, gv, sv, so, Jg, outp, idxp, stats);
            launches += 1;
        } else {
            PairView pv{};
            uint64_t pairs = 0;
            for (int m = 0; m < kMaterials; m++) {
                pv.pairbase[m] = pairs;
                pairs += (uint64_t)(so.matbase[m + 1] - so.matbase[m]) * (uint64_t)g.num_nucs[m];
            }
            grow(g.Lbuf, g.lcap, (int64_t)std::max<uint64_t>(pairs, 1));
            pv.L = g.Lbuf;
            launch_search(g.grid_type, o.search, blocks_for(cn, kSearchTpb, 8 * 4), stream, gv, so, pv);
            XS_CUDA_TRY(cudaEventRecord(g.ev[3], stream));
            launch_interp(blocks_for(cn, kInterpTpb, 4 * 4), stream, gv, so, pv, outp, idxp, stats);
            launches += 2;
        }
        XS_CUDA_TRY(cudaEventRecord(g.ev[4], stream));
        if (host_out) { // D2H on the copy stream, overlapped with the next chunk's kernels
            XS_CUDA_TRY(cudaEventRecord(g.ev_done[buf], stream));
            XS_CUDA_TRY(cudaStreamWaitEvent(g.copy_stream, g.ev_done[buf], 0));
            XS_CUDA_TRY(cudaMemcpyAsync(out_macro + c0 * 5, stage, (size_t)cn * 5 * sizeof(double),
                                        cudaMemcpyDeviceToHost, g.copy_stream));
            XS_CUDA_TRY(cudaEventRecord(g.ev_copied[buf], g.copy_stream));
            copied_pending[buf] = true;
        }
        XS_CUDA_TRY(cudaEventRecord(g.ev[5], stream));
        // timing: a chunk's events are read before the next chunk reuses them; the last
        // chunk's (device-only) times are read after the call's final synchronisation, so
        // timing adds no host round trip inside the last chunk
        const bool last = c0 + chunk >= count;
        if (timing && !(last && !host_out)) {
            XS_CUDA_TRY(cudaStreamSynchronize(stream));
            float a = 0, b = 0, c = 0, d = 0;
            cudaEventElapsedTime(&a, g.ev[1], g.ev[2]);
            cudaEventElapsedTime(&b, g.ev[2], g.ev[4]);
            cudaEventElapsedTime(&c, g.ev[2], g.ev[3]);
            if (host_out) { // timing mode serialises: time the chunk's copy on its own
                XS_CUDA_TRY(cudaStreamSynchronize(g.copy_stream));
                cudaEventRecord(g.ev[5], stream);
                XS_CUDA_TRY(cudaStreamSynchronize(stream));
            }
            cudaEventElapsedTime(&d, g.ev[4], g.ev[5]);
            sample_ms += a;
            lookup_ms += b;
            search_ms += c;
            copy_ms += d;
        }
    }
    for (int b = 0; b < 2; b++) // the call's stream covers every outstanding copy
        if (copied_pending[b])
            XS_CUDA_TRY(cudaStreamWaitEvent(stream, g.ev_copied[b], 0));
    if (!published || count == 0)
        XS_CUDA_TRY(cudaMemcpyAsync(g.stats_h, g.stats_d, 3 * sizeof(uint64_t), cudaMemcpyDeviceToHost, stream));
    XS_CUDA_TRY(cudaEventRecord(g.ev[6], stream));
    XS_CUDA_TRY(cudaStreamSynchronize(stream));
    float total = 0;
    XS_CUDA_TRY(cudaEventElapsedTime(&total, g.ev[0], g.ev[6]));
    if (timing && !host_out && count > 0) { // the last chunk's phases (deferred above)
        float a = 0, b = 0, c = 0;
        cudaEventElapsedTime(&a, g.ev[1], g.ev[2]);
        cudaEventElapsedTime(&b, g.ev[2], g.ev[4]);
        cudaEventElapsedTime(&c, g.ev[2], g.ev[3]);
        sample_ms += a;
        lookup_ms += b;
        search_ms += c;
    }
    if (st) {
        st->hash = g.stats_h[0];
        st->pairs = g.stats_h[1];
        st->lookups = sharded ? g.stats_h[2] : (uint64_t)count;
        st->device_ms = total;
        st->sample_ms = sample_ms;
        st->lookup_ms = lookup_ms;
        st->search_ms = search_ms;
        st->copy_ms = copy_ms;
        st->launches = launches;
    }
}

// xs.h promises synchronous calls: if a launch or copy fails partway through the chunk loop,
// wait for whatever was already queued on the call's stream and the copy stream (ignoring
// their errors) before the error reaches the caller, so no kernel or D2H copy can still write
// into the caller's buffers after the call returned
void run_lookups(Grid &g, int64_t first, int64_t count, uint64_t seed, const xs_opts &o, double *out_macro,
                 int32_t *out_idx, xs_stats *st)
{
    try {
        run_lookups_impl(g, first, count, seed, o, out_macro, out_idx, st);
    } catch (...) {
        cudaStreamSynchronize((cudaStream_t)o.stream);
        if (g.copy_stream)
            cudaStreamSynchronize(g.copy_stream);
        cudaGetLastError();
        throw;
    }
}

void run_sample(Grid &g, int64_t first, int64_t count, uint64_t seed, double *q, int32_t *mat, cudaStream_t s)
{
    if (count == 0)
        return;
    const SampleView sv = make_sample_view(g, seed, first, count);
    k_sample<<<blocks_for(count, 256, 32), 256, 0, s>>>(sv, q, mat);
    XS_CUDA_TRY(cudaGetLastError());
    XS_CUDA_TRY(cudaStreamSynchronize(s));
}

void run_search_points(Grid &g, int64_t count, const double *q, const int32_t *nuc, int search, int32_t *out,
                       cudaStream_t s)
{
    XS_CHECK_ARG(search >= 0 && search < XS_SEARCH_COUNT, "search out of range");
    if (count == 0)
        return;
    SearchPtsFn f = g.grid_type == XS_NUCLIDE     ? pick_pts<XS_NUCLIDE>(search)
                    : g.grid_type == XS_UNIONIZED ? pick_pts<XS_UNIONIZED>(search)
                                                  : pick_pts<XS_HASH>(search);
    f<<<blocks_for(count, 256, 32), 256, 0, s>>>(make_view(g), count, q, nuc, out);
    XS_CUDA_TRY(cudaGetLastError());
    XS_CUDA_TRY(cudaStreamSynchronize(s));
}

} // namespace xs
