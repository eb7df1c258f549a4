// capi.cpp -- the extern "C" boundary declared in include/hdb.h.
// Validation, error state, context lifetime, the sweep scheduler (a12) and the
// Sec. VI planning helpers.  Every entry point converts internal exceptions
// into an hdb_status and a thread-local message.
#include <algorithm>
#include <cmath>
#include <condition_variable>
#include <cstring>
#include <deque>
#include <chrono>
#include <thread>

#include "internal.h"

namespace hdb {
const char* last_error();
extern std::atomic<uint64_t> g_kernel_launches;
}  // namespace hdb

using namespace hdb;

#define HDB_GUARD_BEGIN try {
#define HDB_GUARD_END                  \
    }                                  \
    catch (const hdb::Error& e) {      \
        return e.st;                   \
    }                                  \
    catch (const std::bad_alloc&) {    \
        set_error("host out of memory"); \
        return HDB_ENOMEM;             \
    }                                  \
    catch (...) {                      \
        set_error("internal error");   \
        return HDB_EINTERNAL;          \
    }                                  \
    return HDB_OK;

extern "C" {

const char* hdb_last_error(void) { return hdb::last_error(); }
const char* hdb_version(void) { return "hdb 0.1.0 (sm_100a)"; }

uint64_t hdb_kernel_launches(void) { return g_kernel_launches.load(); }

void hdb_opts_default(hdb_opts* o) {
    if (!o) return;
    memset(o, 0, sizeof *o);
    o->sample_fraction = 0.01;
    o->alpha = 0.05;
    o->n_streams = 3;
}

hdb_status hdb_ctx_create(const hdb_opts* opts, hdb_ctx** out) {
    if (!out) {
        set_error("out is NULL");
        return HDB_EINVAL;
    }
    *out = nullptr;
    hdb_ctx* c = nullptr;
    HDB_GUARD_BEGIN
    hdb_opts o;
    hdb_opts_default(&o);
    if (opts) o = *opts;
    if (!(o.sample_fraction > 0 && o.sample_fraction <= 1)) fail(HDB_EINVAL, "sample_fraction must be in (0,1]");
    if (!(o.alpha >= 0) || !std::isfinite(o.alpha)) fail(HDB_EINVAL, "alpha must be finite and >= 0");
    if (o.n_streams < 1 || o.n_streams > 32) fail(HDB_EINVAL, "n_streams must be in [1,32]");
    if (o.n_devices < 0 || (o.n_devices > 0 && !o.devices)) fail(HDB_EINVAL, "bad device list");
    if (o.shard_count < 0 || (o.shard_count > 0 && (o.shard_rank < 0 || o.shard_rank >= o.shard_count)))
        fail(HDB_EINVAL, "bad shard_rank/shard_count");
    // the search kernels hold 2k+1 <= kMaxSpans row spans per group (kernels_search.cu)
    if (o.cell_split < 0 || o.cell_split > kMaxCellSplit)
        fail(HDB_EINVAL, "cell_split must be in [0, %d]", kMaxCellSplit);
    if (o.sweep_on_device != 0 && o.sweep_on_device != 1) fail(HDB_EINVAL, "sweep_on_device must be 0 or 1");
    c = new hdb_ctx;
    int ndev_avail = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev_avail);
    if (e != cudaSuccess || ndev_avail == 0) {
        cudaGetLastError();
        fail(HDB_ECUDA, "no CUDA device available (%s)", cudaGetErrorString(e));
    }
    if (o.n_devices > 0) {
        c->device_list.assign(o.devices, o.devices + o.n_devices);
    } else {
        int d = 0;
        HDB_CUDA(cudaGetDevice(&d));
        c->device_list.push_back(d);
    }
    for (int d : c->device_list)
        if (d < 0 || d >= ndev_avail) fail(HDB_EINVAL, "device %d out of range", d);
    o.devices = c->device_list.data();
    o.n_devices = (int)c->device_list.size();
    c->opts = o;
    c->pinned = std::make_shared<PinnedPool>();
    int prev = 0;
    cudaGetDevice(&prev);
    for (int d : c->device_list) {
        HDB_CUDA(cudaSetDevice(d));
        DevCtx dc;
        dc.device = d;
        HDB_CUDA(cudaStreamCreateWithFlags(&dc.main, cudaStreamNonBlocking));
        for (int i = 0; i < o.n_streams; ++i) {
            cudaStream_t s;
            HDB_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
            dc.streams.push_back(s);
        }
        HDB_CUDA(cudaHostAlloc((void**)&dc.pin, 256, cudaHostAllocPortable));
        cudaMemPool_t pool;
        HDB_CUDA(cudaDeviceGetDefaultMemPool(&pool, d));
        uint64_t thr = UINT64_MAX;
        HDB_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
        cudaMemPoolProps props{};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = d;
        HDB_CUDA(cudaMemPoolCreate(&dc.big_pool, &props));
        size_t free_b = 0;
        HDB_CUDA(cudaMemGetInfo(&free_b, &dc.total_mem));
        dc.scan_ep.cap = 1u << 20;   // tiles of 4,096 elements: scans of up to 2^32 elements
        HDB_CUDA(cudaMalloc((void**)&dc.scan_ep.tiles, (dc.scan_ep.cap + 1) * sizeof(unsigned long long)));
        HDB_CUDA(cudaMemset(dc.scan_ep.tiles, 0, (dc.scan_ep.cap + 1) * sizeof(unsigned long long)));
        HDB_CUDA(cudaMemPoolSetAttribute(dc.big_pool, cudaMemPoolAttrReleaseThreshold, &thr));
        c->dev.push_back(dc);
    }
    cudaSetDevice(prev);
    *out = c;
    c = nullptr;
    }
    catch (const hdb::Error& err) {
        if (c) hdb_ctx_destroy(c);
        return err.st;
    }
    catch (...) {
        if (c) hdb_ctx_destroy(c);
        set_error("internal error in hdb_ctx_create");
        return HDB_EINTERNAL;
    }
    return HDB_OK;
}

void hdb_ctx_destroy(hdb_ctx* c) {
    if (!c) return;
    int prev = 0;
    cudaGetDevice(&prev);
    for (auto& dc : c->dev) {
        cudaSetDevice(dc.device);
        for (auto s : dc.streams) cudaStreamSynchronize(s);
        if (dc.main) cudaStreamSynchronize(dc.main);
        for (auto* b : dc.batch_buf)
            if (b) cudaFree(b);
        for (auto s : dc.streams) cudaStreamDestroy(s);
        if (dc.main && dc.own_main) cudaStreamDestroy(dc.main);
        if (dc.pin) cudaFreeHost(dc.pin);
        if (dc.scan_ep.tiles) cudaFree(dc.scan_ep.tiles);
        // tables still alive keep their blocks: the pool is then left to process exit
        if (dc.big_pool && c->live_objects == 0) cudaMemPoolDestroy(dc.big_pool);
    }
    cudaSetDevice(prev);
    delete c;
}

hdb_status hdb_ctx_set_stream(hdb_ctx* c, void* stream) {
    if (!c) {
        set_error("ctx is NULL");
        return HDB_EINVAL;
    }
    std::lock_guard<std::recursive_mutex> lk(c->mu);
    HDB_GUARD_BEGIN
    DevCtx& dc = c->dev[0];
    int prev = 0;
    cudaGetDevice(&prev);
    HDB_CUDA(cudaSetDevice(dc.device));
    if (stream) {
        if (dc.own_main) {
            cudaStreamSynchronize(dc.main);
            cudaStreamDestroy(dc.main);
        }
        dc.main = (cudaStream_t)stream;
        dc.own_main = false;
    } else if (!dc.own_main) {
        HDB_CUDA(cudaStreamCreateWithFlags(&dc.main, cudaStreamNonBlocking));
        dc.own_main = true;
    }
    cudaSetDevice(prev);
    HDB_GUARD_END
}

hdb_status hdb_stats_get(const hdb_ctx* c, hdb_stats* out) {
    if (!c || !out) {
        set_error("NULL argument");
        return HDB_EINVAL;
    }
    *out = c->stats;
    return HDB_OK;
}

hdb_status hdb_grid_build(hdb_ctx* c, const void* xy, uint64_t n, hdb_dtype dt, double eps, hdb_grid** out) {
    if (!c || !out) {
        set_error("NULL ctx/out");
        return HDB_EINVAL;
    }
    *out = nullptr;
    std::lock_guard<std::recursive_mutex> lk(c->mu);
    HDB_GUARD_BEGIN
    c->stats = hdb_stats{};
    grid_build(c, xy, n, dt, eps, out);
    HDB_GUARD_END
}

void hdb_grid_free(hdb_grid* g) {
    if (!g) return;
    hdb_ctx* c = g->ctx;
    if (c) {
        std::lock_guard<std::recursive_mutex> lk(c->mu);
        grid_free(g);
    } else {
        grid_free(g);
    }
}

hdb_status hdb_grid_view_get(const hdb_grid* g, hdb_grid_view* v) {
    if (!g || !v) {
        set_error("NULL argument");
        return HDB_EINVAL;
    }
    const DevGrid& d = g->dev[0];
    memset(v, 0, sizeof *v);
    v->n = d.n;
    v->eps = d.eps;
    v->dtype = d.dtype;
    v->xmin = d.xmin;
    v->ymin = d.ymin;
    v->xmax = d.xmax;
    v->ymax = d.ymax;
    v->cell_w = d.w;
    v->nx = d.nx;
    v->ny = d.ny;
    v->n_cells = d.n_cells;
    v->n_nonempty = d.n_nonempty;
    v->n_groups = d.n_groups;
    v->device = d.device;
    v->xy_sorted = d.xy_s;
    v->ids = d.ids;
    v->cell_keys = d.ckey;
    v->cell_start = d.cstart;
    return HDB_OK;
}

hdb_status hdb_grid_copy_to_host(const hdb_grid* g, uint32_t* ids, uint64_t* cell_keys, uint32_t* cell_start,
                                 void* xy_sorted) {
    if (!g) {
        set_error("grid is NULL");
        return HDB_EINVAL;
    }
    HDB_GUARD_BEGIN
    const DevGrid& d = g->dev[0];
    int prev = 0;
    cudaGetDevice(&prev);
    HDB_CUDA(cudaSetDevice(d.device));
    const size_t esz = d.dtype == HDB_F64 ? 16 : 8;
    if (ids && d.n) HDB_CUDA(cudaMemcpy(ids, d.ids, 4 * d.n, cudaMemcpyDeviceToHost));
    if (cell_keys && d.n_nonempty)
        HDB_CUDA(cudaMemcpy(cell_keys, d.ckey, 8 * d.n_nonempty, cudaMemcpyDeviceToHost));
    if (cell_start) HDB_CUDA(cudaMemcpy(cell_start, d.cstart, 4 * (d.n_nonempty + 1), cudaMemcpyDeviceToHost));
    if (xy_sorted && d.n) HDB_CUDA(cudaMemcpy(xy_sorted, d.xy_s, esz * d.n, cudaMemcpyDeviceToHost));
    cudaSetDevice(prev);
    HDB_GUARD_END
}

static hdb_status table_common(hdb_ctx* c, const hdb_grid* g, bool dev, hdb_table** out) {
    if (!c || !g || !out) {
        set_error("NULL argument");
        return HDB_EINVAL;
    }
    *out = nullptr;
    if (g->ctx != c) {
        set_error("grid belongs to another context");
        return HDB_EINVAL;
    }
    std::lock_guard<std::recursive_mutex> lk(c->mu);
    HDB_GUARD_BEGIN
    neighbor_table(c, g, dev, out);
    HDB_GUARD_END
}

hdb_status hdb_neighbor_table(hdb_ctx* c, const hdb_grid* g, hdb_table** out) { return table_common(c, g, false, out); }

hdb_status hdb_neighbor_table_device(hdb_ctx* c, const hdb_grid* g, hdb_table** out) {
    return table_common(c, g, true, out);
}

hdb_status hdb_table_from_host(uint64_t n, const uint64_t* begin, const uint32_t* count, const uint32_t* nbrs,
                               uint64_t npairs, hdb_table** out) {
    if (!out) {
        set_error("out is NULL");
        return HDB_EINVAL;
    }
    *out = nullptr;
    if (n > 0 && (!begin || !count)) {
        set_error("begin/count NULL with n > 0");
        return HDB_EINVAL;
    }
    if (npairs > 0 && !nbrs) {
        set_error("nbrs NULL with npairs > 0");
        return HDB_EINVAL;
    }
    if (n >= 0xffffffffull) {
        set_error("n >= 2^32-1");
        return HDB_ERANGE;
    }
    for (uint64_t p = 0; p < n; ++p) {
        if (begin[p] + count[p] > npairs || begin[p] + count[p] < begin[p]) {
            set_error("row %llu [%llu, +%u) outside nbrs[%llu]", (unsigned long long)p, (unsigned long long)begin[p],
                      count[p], (unsigned long long)npairs);
            return HDB_EINVAL;
        }
    }
    for (uint64_t k = 0; k < npairs; ++k)
        if (nbrs[k] >= n) {
            set_error("nbrs[%llu] = %u >= n", (unsigned long long)k, nbrs[k]);
            return HDB_EINVAL;
        }
    HDB_GUARD_BEGIN
    auto* t = new hdb_table;
    t->n = n;
    t->npairs = npairs;
    t->end_query = n;
    t->malloced = true;
    t->begin = (uint64_t*)malloc(8 * (n ? n : 1));
    t->count = (uint32_t*)malloc(4 * (n ? n : 1));
    t->nbrs = (uint32_t*)malloc(4 * (npairs ? npairs : 1));
    if (!t->begin || !t->count || !t->nbrs) {
        table_free(t);
        fail(HDB_ENOMEM, "host allocation failed");
    }
    if (n) {
        memcpy(t->begin, begin, 8 * n);
        memcpy(t->count, count, 4 * n);
    }
    if (npairs) memcpy(t->nbrs, nbrs, 4 * npairs);
    *out = t;
    HDB_GUARD_END
}

hdb_status hdb_table_view_get(const hdb_table* t, hdb_table_view* v) {
    if (!t || !v) {
        set_error("NULL argument");
        return HDB_EINVAL;
    }
    memset(v, 0, sizeof *v);
    v->n = t->n;
    v->npairs = t->npairs;
    v->begin = t->begin;
    v->count = t->count;
    v->nbrs = t->nbrs;
    v->on_device = t->on_device ? 1 : 0;
    v->device = t->device;
    v->first_query = t->first_query;
    v->end_query = t->end_query;
    v->eps = t->eps;
    v->dtype = t->dtype;
    return HDB_OK;
}

hdb_status hdb_table_copy_to_host(const hdb_table* t, uint64_t* begin, uint32_t* count, uint32_t* nbrs) {
    if (!t) {
        set_error("table is NULL");
        return HDB_EINVAL;
    }
    HDB_GUARD_BEGIN
    if (t->on_device) {
        int prev = 0;
        cudaGetDevice(&prev);
        HDB_CUDA(cudaSetDevice(t->device));
        HDB_CUDA(cudaStreamSynchronize(t->dstream));
        if (begin && t->n) HDB_CUDA(cudaMemcpy(begin, t->begin, 8 * t->n, cudaMemcpyDeviceToHost));
        if (count && t->n) HDB_CUDA(cudaMemcpy(count, t->count, 4 * t->n, cudaMemcpyDeviceToHost));
        if (nbrs && t->npairs) HDB_CUDA(cudaMemcpy(nbrs, t->nbrs, 4 * t->npairs, cudaMemcpyDeviceToHost));
        cudaSetDevice(prev);
    } else {
        if (begin && t->n) memcpy(begin, t->begin, 8 * t->n);
        if (count && t->n) memcpy(count, t->count, 4 * t->n);
        if (nbrs && t->npairs) memcpy(nbrs, t->nbrs, 4 * t->npairs);
    }
    HDB_GUARD_END
}

hdb_status hdb_table_canonicalize(hdb_table* t) {
    if (!t) {
        set_error("table is NULL");
        return HDB_EINVAL;
    }
    if (t->on_device) {
        set_error("hdb_table_canonicalize: table is device-resident");
        return HDB_EINVAL;
    }
    HDB_GUARD_BEGIN
    canonicalize(t);
    HDB_GUARD_END
}

void hdb_table_free(hdb_table* t) {
    if (!t) return;
    table_free(t);
}

hdb_status hdb_dbscan_ex(const hdb_table* t, uint32_t minpts, int n_threads, int32_t* labels, uint8_t* is_core,
                         uint32_t* n_clusters) {
    if (!t) {
        set_error("table is NULL");
        return HDB_EINVAL;
    }
    if (minpts == 0) {
        set_error("minpts must be >= 1");
        return HDB_EINVAL;
    }
    if (t->n > 0 && !labels) {
        set_error("labels is NULL");
        return HDB_EINVAL;
    }
    if (t->first_query != 0 || t->end_query != t->n) {
        set_error("hdb_dbscan: table holds only a shard of the queries");
        return HDB_EINVAL;
    }
    HDB_GUARD_BEGIN
    uint32_t k = 0;
    if (t->on_device) {
        k = dbscan_device(t, minpts, labels, is_core);   // labels / is_core: host or device memory
    } else {
        int T = n_threads > 0 ? n_threads : resolve_threads(t->host_threads);
        k = dbscan_host(t, minpts, T, labels, is_core);
    }
    if (n_clusters) *n_clusters = k;
    HDB_GUARD_END
}

hdb_status hdb_dbscan(const hdb_table* t, uint32_t minpts, int32_t* labels, uint8_t* is_core, uint32_t* n_clusters) {
    return hdb_dbscan_ex(t, minpts, 0, labels, is_core, n_clusters);
}

// ------------------------------------------------------------------ sweep (a12)
// Producer: grid + table for eps_0, eps_1, ... (GPU + D2H).  Consumer: the
// minpts variants of the previous eps, concurrently, on the shared read-only
// table (S3 reuse); the producer builds T(eps_{i+1}) while the
// consumer clusters T(eps_i) (S2 pipelining).  At most two
// tables are resident: the one being clustered and the one being built.
hdb_status hdb_sweep(hdb_ctx* c, const void* xy, uint64_t n, hdb_dtype dt, const double* eps, uint32_t n_eps,
                     const uint32_t* minpts, uint32_t n_minpts, int32_t* labels, uint32_t* n_clusters) {
    if (!c || (n_eps && !eps) || (n_minpts && !minpts) || (n_eps && n_minpts && n && !labels)) {
        set_error("NULL argument");
        return HDB_EINVAL;
    }
    for (uint32_t j = 0; j < n_minpts; ++j)
        if (minpts[j] == 0) {
            set_error("minpts must be >= 1");
            return HDB_EINVAL;
        }
    for (uint32_t i = 0; i < n_eps; ++i)
        if (!std::isfinite(eps[i]) || !(eps[i] > 0)) {
            set_error("eps[%u]=%g must be finite and > 0", i, eps[i]);
            return HDB_EINVAL;
        }
    std::lock_guard<std::recursive_mutex> lk(c->mu);
    HDB_GUARD_BEGIN
    // a process shard builds only its rows of T: clustering it would be silently wrong
    if (c->opts.shard_count > 1) fail(HDB_EINVAL, "hdb_sweep needs an unsharded context (shard_count <= 1)");
    if (c->opts.sweep_on_device) {
        // NEXT-4 variant: T(eps_i) stays in HBM; every minpts variant runs the
        // device DBSCAN on it and only labels cross PCIe.
        for (uint32_t i = 0; i < n_eps; ++i) {
            hdb_grid* g = nullptr;
            hdb_table* t = nullptr;
            try {
                grid_build(c, xy, n, dt, eps[i], &g);
                neighbor_table(c, g, true, &t, /*pos_space=*/true);   // internal: clustered in position space
                grid_free(g);
                g = nullptr;
                for (uint32_t j = 0; j < n_minpts; ++j) {
                    const uint32_t k = dbscan_device(t, minpts[j], labels + ((uint64_t)i * n_minpts + j) * n, nullptr);
                    if (n_clusters) n_clusters[(uint64_t)i * n_minpts + j] = k;
                }
                table_free(t);
            } catch (...) {
                if (g) grid_free(g);
                if (t) table_free(t);
                throw;
            }
        }
        return HDB_OK;
    }
    if (n && n_eps && n_minpts && is_device_ptr(labels))
        fail(HDB_EINVAL, "hdb_sweep: labels must be host memory unless opts.sweep_on_device = 1");
    std::mutex m;
    std::condition_variable cv;
    std::deque<std::pair<uint32_t, hdb_table*>> q;
    bool slot_free = true;   // producer may build only while the queue is empty
    bool done = false;
    hdb_status prod_st = HDB_OK;
    std::string prod_msg;
    int dev0 = c->dev[0].device;
    // HDB_TIMELINE=1: host timeline of the pipeline (ms from the call's start) as one JSON
    // line on stderr -- the overlap of T(eps_{i+1})'s build with T(eps_i)'s clustering
    const char* tle = getenv("HDB_TIMELINE");
    const bool tl = tle && *tle == '1';
    const auto t_start = std::chrono::steady_clock::now();
    auto now_ms = [&] {
        return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count();
    };
    std::vector<double> tb0(n_eps, 0), tb1(n_eps, 0), tc0(n_eps, 0), tc1(n_eps, 0);
    std::thread producer([&] {
        cudaSetDevice(dev0);
        for (uint32_t i = 0; i < n_eps; ++i) {
            {
                std::unique_lock<std::mutex> l(m);
                cv.wait(l, [&] { return slot_free || done; });
                if (done) return;   // the consumer stopped (a DBSCAN variant failed)
                slot_free = false;
            }
            hdb_grid* g = nullptr;
            hdb_table* t = nullptr;
            try {
                tb0[i] = now_ms();
                grid_build(c, xy, n, dt, eps[i], &g);
                neighbor_table(c, g, false, &t);
                grid_free(g);
                tb1[i] = now_ms();
            } catch (const hdb::Error& e) {
                if (g) grid_free(g);
                std::lock_guard<std::mutex> l(m);
                prod_st = e.st;
                prod_msg = last_error();
                done = true;
                cv.notify_all();
                return;
            } catch (...) {
                if (g) grid_free(g);
                std::lock_guard<std::mutex> l(m);
                prod_st = HDB_EINTERNAL;
                prod_msg = "internal error in sweep producer";
                done = true;
                cv.notify_all();
                return;
            }
            std::lock_guard<std::mutex> l(m);
            q.emplace_back(i, t);
            cv.notify_all();
        }
        std::lock_guard<std::mutex> l(m);
        done = true;
        cv.notify_all();
    });
    const int T = resolve_threads(c->opts.host_threads);
    const int per = std::max(1, T / (int)std::max<uint32_t>(1, n_minpts));
    for (uint32_t got = 0; got < n_eps; ++got) {
        std::pair<uint32_t, hdb_table*> item{0, nullptr};
        {
            std::unique_lock<std::mutex> l(m);
            cv.wait(l, [&] { return !q.empty() || done; });
            if (q.empty()) break;   // producer failed
            item = q.front();
            q.pop_front();
            slot_free = true;       // let the producer build the next table now
            cv.notify_all();
        }
        const uint32_t i = item.first;
        hdb_table* t = item.second;
        tc0[i] = now_ms();
        std::vector<std::thread> th;
        std::vector<hdb_status> st(n_minpts, HDB_OK);
        for (uint32_t j = 0; j < n_minpts; ++j)
            th.emplace_back([&, j] {
                uint32_t k = 0;
                try {
                    k = dbscan_host(t, minpts[j], per, labels + ((uint64_t)i * n_minpts + j) * n, nullptr);
                } catch (...) {
                    st[j] = HDB_ENOMEM;
                }
                if (n_clusters) n_clusters[(uint64_t)i * n_minpts + j] = k;
            });
        for (auto& x : th) x.join();
        tc1[i] = now_ms();
        table_free(t);
        for (auto s : st)
            if (s != HDB_OK) {
                {
                    std::lock_guard<std::mutex> l(m);
                    done = true;
                    cv.notify_all();
                }
                producer.join();
                // tables the producer queued meanwhile are freed before reporting
                while (!q.empty()) {
                    table_free(q.front().second);
                    q.pop_front();
                }
                fail(s, "sweep: DBSCAN variant failed");
            }
    }
    producer.join();
    {
        std::lock_guard<std::mutex> l(m);
        while (!q.empty()) {
            table_free(q.front().second);
            q.pop_front();
        }
    }
    if (tl) {
        std::string js = "{\"timeline\": \"hdb_sweep\", \"total_ms\": " + std::to_string(now_ms()) + ", \"eps\": [";
        for (uint32_t i = 0; i < n_eps; ++i) {
            char b[256];
            snprintf(b, sizeof b, "%s{\"eps\": %g, \"build\": [%.3f, %.3f], \"dbscan\": [%.3f, %.3f]}", i ? ", " : "",
                     eps[i], tb0[i], tb1[i], tc0[i], tc1[i]);
            js += b;
        }
        js += "]}";
        fprintf(stderr, "%s\n", js.c_str());
    }
    if (prod_st != HDB_OK) {
        set_error("%s", prod_msg.c_str());
        return prod_st;
    }
    HDB_GUARD_END
}

// ------------------------------------------------------------------ Sec. VI helpers
hdb_status hdb_plan_batches(double est_pairs, double alpha, int n_streams, double* b_b, uint64_t* n_b) {
    if (!(est_pairs >= 0) || !(alpha >= 0) || n_streams < 1 || !b_b || !n_b) {
        set_error("bad argument to hdb_plan_batches");
        return HDB_EINVAL;
    }
    // buffer rule (reading R13: threshold on the total estimate,
    // 3e8 = 3 streams x 1e8): fixed 1e8 pairs per stream for large results,
    // else est * (1 + 2 alpha) / n_streams.
    const double thresh = 1e8 * n_streams;
    double bb = est_pairs >= thresh ? 1e8 : est_pairs * (1.0 + 2.0 * alpha) / n_streams;
    if (bb < 1) bb = 1;
    *b_b = bb;
    // Eq. 1: n_b = ceil((1 + alpha) a_b / b_b)
    double nb = std::ceil((1.0 + alpha) * est_pairs / bb);
    *n_b = (uint64_t)std::max(1.0, nb);
    return HDB_OK;
}

uint64_t hdb_strided_point(uint64_t gid, uint64_t l, uint64_t n_b) { return gid * n_b + l; }

hdb_status hdb_balanced_cuts(const uint64_t* prefix, uint64_t n_items, uint32_t parts, uint64_t* cuts) {
    if (!prefix || !cuts || parts == 0) {
        set_error("bad argument to hdb_balanced_cuts");
        return HDB_EINVAL;
    }
    const uint64_t total = prefix[n_items];
    cuts[0] = 0;
    for (uint32_t k = 1; k < parts; ++k) {
        const uint64_t target = (uint64_t)(((unsigned __int128)total * k) / parts);
        // first item index i with prefix[i] >= target (cut before item i)
        const uint64_t* it = std::lower_bound(prefix, prefix + n_items + 1, target);
        uint64_t i = (uint64_t)(it - prefix);
        if (i > n_items) i = n_items;
        // take the nearer of the two prefix boundaries around the target
        if (i > 0 && target - prefix[i - 1] < (i <= n_items ? prefix[i] - target : ~0ull)) --i;
        cuts[k] = std::max(cuts[k - 1], i);
    }
    cuts[parts] = n_items;
    return HDB_OK;
}

}  // extern "C"
