// engine.cpp -- host orchestration of the hot path.
//
//   grid_build      a1-a4 on every device of the context (each holds the full
//                   point set and its grid).
//   neighbor_table  a5 sampled count + plan (Sec. VI, Eq. 1 P:736-741,
//                   buffer rule P:812-823), query shards (devices x processes),
//                   a6 exact count, a7 scan, the "final gather of counts" that
//                   gives every shard its base offset, a8 batched write kernels
//                   round-robin over n_streams streams with each
//                   batch DMA'd straight into the host table (a9/a10: the
//                   paper's T_i^min/max + B layout, without the
//                   pinned->pageable staging copy), or a device-resident table.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <exception>
#include <memory>
#include <thread>

#include "internal.h"

namespace hdb {

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;

void set_error(const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
}

void fail(hdb_status st, const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    throw Error{st};
}

const char* last_error() { return g_err.c_str(); }

int resolve_threads(int req) {
    if (req > 0) return req;
    unsigned h = std::thread::hardware_concurrency();
    return h ? (int)h : 1;
}

// ------------------------------------------------------------------ pools
void* PinnedPool::acquire(size_t bytes, size_t* got) {
    std::lock_guard<std::mutex> lk(m);
    if (bytes == 0) bytes = 64;
    auto it = free_blocks.lower_bound(bytes);
    if (it != free_blocks.end() && it->first <= 2 * bytes + (64u << 20)) {
        void* p = it->second;
        *got = it->first;
        free_blocks.erase(it);
        return p;
    }
    size_t sz = (bytes + (2u << 20) - 1) & ~(size_t)((2u << 20) - 1);
    void* p = nullptr;
    cudaError_t e = cudaHostAlloc(&p, sz, cudaHostAllocPortable);
    if (e != cudaSuccess) {
        cudaGetLastError();
        for (auto& kv : free_blocks) {
            cudaFreeHost(kv.second);
            bytes_total -= kv.first;
        }
        free_blocks.clear();
        e = cudaHostAlloc(&p, sz, cudaHostAllocPortable);
        if (e != cudaSuccess) {
            cudaGetLastError();
            fail(HDB_ENOMEM, "pinned host allocation of %zu bytes failed: %s", sz, cudaGetErrorString(e));
        }
    }
    bytes_total += sz;
    ++grows;
    *got = sz;
    return p;
}

void PinnedPool::release(void* p, size_t bytes) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(m);
    free_blocks.emplace(bytes, p);
}

PinnedPool::~PinnedPool() {
    for (auto& kv : free_blocks) cudaFreeHost(kv.second);
}

// ------------------------------------------------------------------ helpers
namespace {

// HDB_TRACE=1: host wall-clock marks of the phases of each call, to stderr.
struct Trace {
    bool on = false;
    const char* what;
    std::chrono::steady_clock::time_point t0, last;
    std::string buf;
    explicit Trace(const char* w) : what(w) {
        const char* e = getenv("HDB_TRACE");
        on = e && *e == '1';
        t0 = last = std::chrono::steady_clock::now();
    }
    void mark(const char* name) {
        if (!on) return;
        auto t = std::chrono::steady_clock::now();
        char b[96];
        snprintf(b, sizeof b, " %s=%.3f", name, std::chrono::duration<double, std::milli>(t - last).count());
        buf += b;
        last = t;
    }
    ~Trace() {
        if (on)
            fprintf(stderr, "[hdb trace] %s total=%.3f ms:%s\n", what,
                    std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count(),
                    buf.c_str());
    }
};

// HDB_TIMELINE=1: the batched host-table write (a8 + a9) prints its GPU timeline as
// one JSON line to stderr -- per batch, the write kernel's and the D2H copy's start / end
// (CUDA events, ms from the first batch) and stream -- the overlap evidence of P:796-812
bool timeline_on() {
    static const bool on = [] {
        const char* e = getenv("HDB_TIMELINE");
        return e && *e == '1';
    }();
    return on;
}

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int d) {
        cudaGetDevice(&prev);
        if (prev != d) HDB_CUDA(cudaSetDevice(d));
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

// stream-ordered device buffer, freed at scope exit unless released
struct DBuf {
    void* p = nullptr;
    cudaStream_t s = nullptr;
    DBuf() = default;
    // pool: the device's big_pool for table-sized buffers (null = the default pool)
    DBuf(size_t bytes, cudaStream_t st, cudaMemPool_t pool = nullptr) : s(st) {
        if (bytes == 0) bytes = 16;
        cudaError_t e = pool ? cudaMallocFromPoolAsync(&p, bytes, pool, st) : cudaMallocAsync(&p, bytes, st);
        if (e != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
            fail(HDB_ENOMEM, "device allocation of %zu bytes failed: %s", bytes, cudaGetErrorString(e));
        }
    }
    DBuf(const DBuf&) = delete;
    DBuf& operator=(const DBuf&) = delete;
    DBuf(DBuf&& o) noexcept : p(o.p), s(o.s) { o.p = nullptr; }
    DBuf& operator=(DBuf&& o) noexcept {
        reset();
        p = o.p;
        s = o.s;
        o.p = nullptr;
        return *this;
    }
    ~DBuf() { reset(); }
    void reset() {
        if (p) cudaFreeAsync(p, s);
        p = nullptr;
    }
    void* release() {
        void* q = p;
        p = nullptr;
        return q;
    }
    template <typename T>
    T* as() const {
        return (T*)p;
    }
};

struct Event {
    cudaEvent_t e = nullptr;
    Event() { HDB_CUDA(cudaEventCreate(&e)); }
    ~Event() {
        if (e) cudaEventDestroy(e);
    }
    Event(const Event&) = delete;
    Event& operator=(const Event&) = delete;
};

float elapsed(const Event& a, const Event& b) {
    float ms = 0;
    HDB_CUDA(cudaEventElapsedTime(&ms, a.e, b.e));
    return ms;
}

constexpr uint64_t kMaxCellsAbs = 1ull << 30;

// Dense/sparse split (NEXT-1): a query group goes to the thread-per-query kernel
// when (queries x candidates) <= this many tests (
// HDB_SPARSE_TESTS overrides it for tuning, 0 disables the split).
constexpr double kSparseMinShare = 0.25;   // split only when >= this share of the queries is sparse
// Device-resident whole tables take the single-pass kernel (k_fused: count,
// reserve, emit and T by id per group; heavy groups first) unless the
// dense/sparse split is on or the sampled estimate says < this many pairs per
// query.  Measured on one B200 (ms per step, two passes vs single pass, both
// writing T by id): C2 eps 0.15 (97 pairs per query) 1.40 vs 1.25, eps 0.45
// (709) 2.39 vs 2.10 (table kernels), eps 1.40 (4,600) 13.1 vs 9.8 (table
// kernels); C5 (80) 23.1 vs 21.5.  The count work hides under the store stream.
constexpr double kFusedMinPairsPerQuery = 20.0;
// ... and without any sample when the grid's candidate tests per query are clearly in the
// single pass's regime (C2 eps 0.15: 245, eps 0.45: 1,128, eps 1.40: 6,280; C5: 224) and
// 4 B per test fits in this share of the device memory
constexpr double kFusedDirectTestsPerQuery = 150.0;
constexpr double kFusedDirectMemShare = 0.3;
// Query-lane classification (k_qlanes): small groups' queries one
// per lane.  Default: on for point sets beyond the L2 -- the regime in which k_fused visits
// groups in the natural order (coordinates + ids > 256 MB, use_cost_order), where the warp
// per 11-query group of C5's sparse area is latency-bound; below it (C2 eps 0.15, C3, C1)
// k_fused / k_sparse_fused stay faster (profiles/r2x).  HDB_QLANES=1 / 0 forces it on / off.
bool qlanes_enabled(uint64_t n, hdb_dtype dt) {   // read per grid build (tests switch it within one process)
    const char* e = std::getenv("HDB_QLANES");
    if (e && *e) return std::strtol(e, nullptr, 10) != 0;
    const uint64_t esz = dt == HDB_F64 ? 16 : 8;
    return n * (esz + 4) > (256ull << 20);
}
uint32_t sparse_max_tests() {
    static const uint32_t v = [] {
        const char* e = std::getenv("HDB_SPARSE_TESTS");
        return e ? (uint32_t)std::strtoul(e, nullptr, 10) : 256u;
    }();
    return v;
}

enum class Loc { Host, Device };

struct PtrInfo {
    Loc loc = Loc::Host;
    int device = -1;
};

PtrInfo classify(const void* p) {
    PtrInfo r;
    if (!p) return r;
    cudaPointerAttributes a{};
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return r;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
        r.loc = Loc::Device;
        r.device = a.device;
    }
    return r;
}

}  // namespace

bool is_device_ptr(const void* p) { return classify(p).loc == Loc::Device; }

namespace {

// f64 mode: bound on |t_f32 - (d2_f64 - e2_f64)| for the search kernels' f32
// filter.  Filter coordinates are X = fl32(fl64(x - o))
// for an origin o with |x - o| <= R; every candidate lies in the 3x3 stencil,
// so |x_p - x_q| < Dmax = 2w.  With u = 2^-24:
//   E     = R (u + 2^-52)                    (|X - (x - o)|)
//   delta = 2E + (Dmax + 2E) u               (|fl32(X_p - X_q) - (x_p - x_q)|)
//   |t - S| <= 2 delta (2 Dmax + delta)      (the two squares)
//            + u (e2 + (Dmax^2 + e2) + (2 Dmax^2 + e2)) (1 + 2^-20)   (e2 rounding, 2 fma roundings)
//            + 2^-49 Dmax^2                  (the f64 predicate's own rounding)
// and the kernels use band = 2x that bound (rounded up): |t| > band => sign(t)
// is the exact f64 decision.  Two origins are used:
//   * count pass (k_count): o = the group's first query, R = Dmax (local, tiny band,
//     so band tests are detected per chunk, ~1e-3 of chunks);
//   * recompute write variant: o = bbox centre, R = bbox half-extent.
// A filter is disabled (exact f64 kernel) when float overflow is possible or its
// band would cover a large part of eps^2.
static double filter_band(double R, double Dmax, double e2) {
    const double u = 0x1p-24;
    const double E = R * (u + 0x1p-52);
    const double delta = 2 * E + (Dmax + 2 * E) * u;
    const double bound = 2 * delta * (2 * Dmax + delta) + u * (3 * e2 + 3 * Dmax * Dmax) * (1 + 0x1p-20) +
                         0x1p-49 * Dmax * Dmax;
    return 2.0 * bound;
}

static float round_up_f(double v) {
    float f = (float)v;
    if ((double)f < v) f = std::nextafter(f, INFINITY);
    return f;
}

void set_filter_bound(DevGrid& g) {
    g.filter = g.filter_l = g.filter_b = false;
    g.band = g.band_l = 0;
    g.nb2_l = g.nb2_b = 0;
    if (g.dtype != HDB_F64) return;
    g.ox = 0.5 * g.xmin + 0.5 * g.xmax;
    g.oy = 0.5 * g.ymin + 0.5 * g.ymax;
    const double R = std::max(std::max(std::fabs(g.xmax - g.ox), std::fabs(g.xmin - g.ox)),
                              std::max(std::fabs(g.ymax - g.oy), std::fabs(g.ymin - g.oy)));
    // stencil of +-k cells: |x_p - x_q| < (k+1) w; cell rounding adds <= 2^-21 cell widths
    const double Dmax = (double)(g.split + 1) * g.w * (1.0 + 0x1p-18);
    const double e2 = g.e2_d;
    g.e2_f = (float)e2;
    if (!(Dmax < 1e15) || !(e2 > 1e-30)) return;
    const double band = filter_band(R, Dmax, e2);
    if (R < 1e15 && band < 0.25 * e2) {
        g.band = round_up_f(band);
        g.filter = true;
    }
    // query-lane blocks: coordinates relative to the block's first query, queries and staged
    // candidates within kQCX + k + 1 cell widths of it (x) and k + 1 (y)
    const double Rb = ((double)kQCX + (double)g.split + 1.0) * g.w * (1.0 + 0x1p-18);
    const double band_b = filter_band(Rb, Dmax, e2);
    if (Rb < 1e15 && band_b < 0.25 * e2) {
        const double B = band_b * (1.0 + 0x1p-20);
        g.nb2_b = -round_up_f(B * B);
        g.filter_b = true;
    }
    const double band_l = filter_band(Dmax, Dmax, e2);
    if (band_l < 0.25 * e2) {
        // flag test in the kernel: fma(t, t, -B^2) < 0 with B = band_l (1 + 2^-20) covers |t| <= band_l
        const double B = band_l * (1.0 + 0x1p-20);
        g.band_l = round_up_f(band_l);
        g.nb2_l = -round_up_f(B * B);
        g.filter_l = true;
    }
}

// Default cell split (hdb_opts.cell_split == 0; split_from_occ): cells of width eps/k with
// k = floor(sqrt(occ / 25)) clamped to [1, 6], where occ = sum n_c (n_c - 1) / n is
// the point-weighted occupancy of the eps-wide cells, estimated from a strided
// sample of <= 8192 points.  Finer cells shrink each group's candidate region
// ((2 + 1/k)^2 eps^2 instead of 9 eps^2) but make groups smaller; ~25 points
// per split cell was the measured break-even on the C2/C3 stand-ins.
constexpr uint32_t kOccTable = 1u << 15;
constexpr uint64_t kOccSample = 8192;

uint32_t split_from_occ(const unsigned long long* h, uint64_t n, const DevGrid& g, double eps_used) {
    if (h[1] == 0) return 1;
    const uint64_t m = std::min<uint64_t>(n, kOccSample);
    const double f = (double)m / (double)n;
    const double occ = (double)h[0] / (f * (double)h[1]);
    uint32_t k = (uint32_t)std::floor(std::sqrt(occ / 25.0));
    k = std::max<uint32_t>(1, std::min<uint32_t>(k, 6));
    const double inv1 = 1.0 / (eps_used * (1.0 + 0x1p-19));
    const double ex = (g.xmax - g.xmin) * inv1, ey = (g.ymax - g.ymin) * inv1;
    while (k > 1 && (ex * k > 0x1p30 || ey * k > 0x1p30)) --k;
    return k;
}

constexpr double kPointPairs = 117.0;   // a query's fixed work in pair-equivalents (band weights)

// HDB_BANDS=0 turns the process-shard bands off (every rank then builds the full grid)
bool bands_enabled() {
    static const bool on = [] {
        const char* e = std::getenv("HDB_BANDS");
        return !(e && *e == '0');
    }();
    return on;
}

// rows [y0, y1) of shard `rank` of R: the cut rows split the cumulative load into R
// equal parts (cut r = first row whose prefix load reaches r/R of the total)
void band_rows(const std::vector<uint64_t>& load, uint32_t R, uint32_t rank, uint64_t& y0, uint64_t& y1) {
    const uint64_t ny = load.size();
    unsigned __int128 total = 0;
    for (uint64_t v : load) total += v;
    auto cut = [&](uint32_t r) -> uint64_t {
        if (r == 0) return 0;
        if (r >= R) return ny;
        const unsigned __int128 target = total * r / R;
        unsigned __int128 acc = 0;
        for (uint64_t y = 0; y < ny; ++y) {
            if (acc >= target) return y;
            acc += load[y];
        }
        return ny;
    };
    y0 = cut(rank);
    y1 = std::max(y0, cut(rank + 1));
}

void build_dev(hdb_ctx* ctx, DevCtx& dc, const void* xy, PtrInfo where, uint64_t n_in, hdb_dtype dt, double eps,
               DevGrid& g) {
    DeviceGuard dg(dc.device);
    cudaStream_t s = dc.main;
    const size_t esz = dt == HDB_F64 ? 16 : 8;
    uint64_t n = n_in;   // points of this grid (a process shard's band: fewer than the input's)
    g.device = dc.device;
    g.dtype = dt;
    g.n = n;
    g.n_ids = n_in;
    g.stream = s;
    Event ev0, ev1;
    HDB_CUDA(cudaEventRecord(ev0.e, s));

    Trace tr("grid_build");
    ScanEpochScope scan_scope(&dc.scan_ep);   // the build's scans: no status memsets
    // ---- a1: ingest + bbox + validation
    DBuf xin_owned;
    const void* xin = xy;
    if (n > 0) {
        if (where.loc == Loc::Host) {
            xin_owned = DBuf(n * esz, s);
            HDB_CUDA(cudaMemcpyAsync(xin_owned.p, xy, n * esz, cudaMemcpyHostToDevice, s));
            __atomic_fetch_add(&ctx->stats.bytes_h2d, (uint64_t)(n * esz), __ATOMIC_RELAXED);   // devices build in parallel
            xin = xin_owned.p;
        } else if (where.device != dc.device) {
            xin_owned = DBuf(n * esz, s);
            HDB_CUDA(cudaMemcpyPeerAsync(xin_owned.p, dc.device, xy, where.device, n * esz, s));
            xin = xin_owned.p;
        }
    }
    // misc (1 KB, zeroed by the bbox init except the bbox sentinels): [0..3] bbox, [4] nonempty,
    // [5] bad count, [6..7] occupancy sums, [8..9] sparse queries / candidate tests,
    // [16..21] readbacks of the group phase, [32..95] cost-order histogram + cursors
    constexpr uint32_t kMiscWords = 128;
    DBuf misc(8 * kMiscWords, s);
    unsigned long long* bb = misc.as<unsigned long long>();
    unsigned int* bad = (unsigned int*)(bb + 5);
    // default cell split: occupancy estimate launched with the bbox, read in the same sync
    const bool auto_k = ctx->opts.cell_split == 0 && n >= 4096;
    DBuf hk, hc;
    if (auto_k) {
        hk = DBuf(8ull * kOccTable, s);
        hc = DBuf(4ull * kOccTable, s);
    }
    launch_bbox_init(bb, kMiscWords, hk.as<unsigned long long>(), hc.as<unsigned int>(), auto_k ? kOccTable : 0, s);
    launch_bbox(xin, n, dt, bb, bad, s);
    HDB_LAUNCH_CHECK();
    tr.mark("bbox-enqueue");
    // small readbacks go through the context's pinned scratch (pin[10..23]): a D2H copy
    // into pageable memory is synchronous and cost ~30 us each here
    unsigned long long* hb = (unsigned long long*)dc.pin + 10;   // bb[0..7] -> pin[10..17]
    const unsigned long long* hocc = hb + 6;
    if (auto_k) {
        const double eps_pre = dt == HDB_F32 ? (double)(float)eps : eps;
        const uint64_t m = std::min<uint64_t>(n, kOccSample);
        launch_occ_estimate(xin, n, dt, n / m, m, 1.0 / (eps_pre * (1.0 + 0x1p-19)), hk.as<unsigned long long>(),
                            hc.as<unsigned int>(), kOccTable, bb + 6, s);
        HDB_LAUNCH_CHECK();
    }
    HDB_CUDA(cudaMemcpyAsync(hb, bb, 64, cudaMemcpyDeviceToHost, s));
    tr.mark("occ-enqueue");
    HDB_CUDA(cudaStreamSynchronize(s));
    hk.reset();
    hc.reset();
    if ((unsigned int)hb[5] != 0) fail(HDB_EINVAL, "%u non-finite coordinate(s)", (unsigned)hb[5]);

    double eps_used = eps;
    if (dt == HDB_F32) {
        float ef = (float)eps;
        if (!(ef > 0.0f) || !std::isfinite(ef)) fail(HDB_EINVAL, "eps=%g is not a positive finite float", eps);
        eps_used = (double)ef;
        g.e2_f = ef * ef;               // fl32(eps_f * eps_f)
    }
    g.e2_d = eps_used * eps_used;       // fl64(eps * eps)
    g.eps = eps_used;
    if (n > 0) {
        g.xmin = bbox_decode(hb[0], false);
        g.ymin = bbox_decode(hb[1], false);
        g.xmax = bbox_decode(hb[2], true);
        g.ymax = bbox_decode(hb[3], true);
    }
    // reading R9: w = eps_F (1 + 2^-19) / k; a neighbour is at most k cells away
    g.split = (uint32_t)(ctx->opts.cell_split > 0 ? ctx->opts.cell_split : 1);
    if (auto_k) g.split = split_from_occ(hocc, n, g, eps_used);
    g.nspan = 2 * g.split + 1;
    g.w = eps_used * (1.0 + 0x1p-19) / (double)g.split;
    g.inv_w = 1.0 / g.w;
    const double ex = (g.xmax - g.xmin) * g.inv_w;   // same rounded ops as the key kernel
    const double ey = (g.ymax - g.ymin) * g.inv_w;
    if (!(ex <= 0x1p30) || !(ey <= 0x1p30))
        fail(HDB_ERANGE, "extent/eps too large (%g x %g cells > 2^30)", ex, ey);
    g.nx = (uint32_t)std::floor(ex) + 1;
    g.ny = (uint32_t)std::floor(ey) + 1;
    g.n_cells = (uint64_t)g.nx * g.ny;   // < 2^61: only the non-empty ones are stored
    set_filter_bound(g);

    tr.mark("bbox+sync");
    // ---- process shard (torchrun rank r of R, one device): a band of cell rows as queries
    // plus k halo rows of candidates on either side -- only those points are sorted (the
    // grid build is not replicated across ranks)
    DBuf band_pts, band_gid;
    uint64_t band_y0 = 0, band_y1 = 0;
    const uint32_t R_proc = ctx->opts.shard_count > 0 ? (uint32_t)ctx->opts.shard_count : 1;
    if (R_proc > 1 && ctx->dev.size() == 1 && n > 0 && g.ny <= (1u << 22) && bands_enabled()) {
        const uint32_t rank = (uint32_t)ctx->opts.shard_rank;
        const bool dense = g.n_cells <= std::max<uint64_t>(8 * n, 1ull << 22);
        DBuf rc(8ull * g.ny, s), rl(8ull * g.ny, s), cc, rowid(4 * n, s);
        HDB_CUDA(cudaMemsetAsync(rc.p, 0, 8ull * g.ny, s));
        HDB_CUDA(cudaMemsetAsync(rl.p, 0, 8ull * g.ny, s));
        if (dense) {
            cc = DBuf(4 * g.n_cells, s);
            HDB_CUDA(cudaMemsetAsync(cc.p, 0, 4 * g.n_cells, s));
        }
        band_rows_hist(xin, n, dt, g.xmin, g.ymin, g.inv_w, g.nx, g.ny, rowid.as<uint32_t>(), cc.as<uint32_t>(),
                       rc.as<unsigned long long>(), rl.as<unsigned long long>(), s);
        HDB_LAUNCH_CHECK();
        cc.reset();
        std::vector<uint64_t> hrc(g.ny), hrl(g.ny);
        HDB_CUDA(cudaMemcpyAsync(hrc.data(), rc.p, 8ull * g.ny, cudaMemcpyDeviceToHost, s));
        HDB_CUDA(cudaMemcpyAsync(hrl.data(), rl.p, 8ull * g.ny, cudaMemcpyDeviceToHost, s));
        HDB_CUDA(cudaStreamSynchronize(s));
        // row weight = estimated pairs + a per-point cost in pair-equivalents.  A cell of m
        // points (width eps/k, locally uniform density) has queries with ~pi k^2 m neighbours
        // each, so a row's pairs ~ pi k^2 sum m^2; and a query costs ~117 pairs' worth of time
        // beside its pairs (least squares over the per-rank steps of C5 at R = 4 and 8:
        // 1.49 ms per rank + 0.187 ms per M points + 0.0016 ms per M pairs -- the grid build
        // and the per-group set-up are per point)
        std::vector<uint64_t> load(g.ny);
        const double kk = 3.14159265358979 * (double)g.split * (double)g.split / 256.0;
        for (uint64_t y = 0; y < g.ny; ++y)
            load[y] = (uint64_t)((dense ? kk * (double)hrl[y] : 0.0) + kPointPairs * (double)hrc[y]);
        band_rows(load, R_proc, rank, band_y0, band_y1);
        const uint64_t ylo = band_y0 >= g.split ? band_y0 - g.split : 0;
        const uint64_t yhi = std::min<uint64_t>(g.ny, band_y1 + g.split);
        uint64_t q0 = 0, q1 = 0, nb = 0;
        for (uint64_t y = 0; y < g.ny; ++y) {
            if (y < band_y0) q0 += hrc[y];
            if (y < band_y1) q1 += hrc[y];
            if (y >= ylo && y < yhi) nb += hrc[y];
        }
        band_pts = DBuf(esz * (nb ? nb : 1), s);
        band_gid = DBuf(4 * (nb ? nb : 1), s);
        DBuf dnb(8, s), btemp(scan_temp_bytes(n + 1), s);
        band_select(xin, rowid.as<uint32_t>(), n, dt, ylo, yhi, band_pts.p, band_gid.as<uint32_t>(),
                    dnb.as<uint32_t>(), btemp.p, s);
        HDB_LAUNCH_CHECK();
        xin = band_pts.p;
        n = nb;
        g.n = n;
        g.banded = true;
        g.band_q0 = q0;
        g.band_q1 = q1;
        tr.mark("band");
    }
    // ---- a2 + a3: the points sorted by cell key (record radix sort over only the bits the
    // key range needs; the first pass computes the keys from the input points, the last
    // writes A, the sorted points and the f32 filter copy -- no separate gather).  ids and
    // points are padded by 2 entries: the search kernels load candidate pairs (2k, 2k+1)
    // with one vector load and mask the invalid half
    const int kb = g.n_cells <= (1ull << 32) ? 4 : 8;   // 32-bit keys whenever they fit
    int bits = 1;
    while (bits < 64 && (1ull << bits) < g.n_cells) ++bits;
    DBuf keys(kb * (n ? n : 1), s), ids(4 * (n + 2), s);
    DBuf xy_s((n + 2) * esz, s);
    DBuf xp(16 * (n / 2 + 2), s);
    DBuf counters(4 * kCounterSlots, s);
    if (n > 0) {
        DBuf stemp(point_sort_temp_bytes(n, dt, kb, bits), s);   // stream-ordered: freed after the sort
        sort_points(xin, n, dt, g.xmin, g.ymin, g.inv_w, g.nx, g.ny, kb, bits, keys.p, ids.as<uint32_t>(), xy_s.p,
                    xp.as<float4>(), g.ox, g.oy, counters.as<unsigned int>(), kCounterSlots, stemp.p, s,
                    g.banded ? band_gid.as<uint32_t>() : nullptr);
        HDB_LAUNCH_CHECK();
    } else {
        HDB_CUDA(cudaMemsetAsync(ids.p, 0, 8, s));
        HDB_CUDA(cudaMemsetAsync(xy_s.p, 0, 2 * esz, s));
        HDB_CUDA(cudaMemsetAsync(xp.p, 0, 32, s));
        HDB_CUDA(cudaMemsetAsync(counters.p, 0, 4 * kCounterSlots, s));
    }
    xin_owned.reset();
    band_pts.reset();
    band_gid.reset();
    DBuf temp(scan_temp_bytes(n + 1), s);
    tr.mark("sort(enqueue)");
    // ---- a4: run-length encoding of the sorted keys -> (key, start) of the non-empty cells
    // (one scan kernel; the arrays are sized by n, the cell count is read back)
    DBuf ckey(8 * (n ? n : 1), s), cstart(4 * (n + 1), s);
    uint32_t* hne_p = (uint32_t*)(dc.pin + 26);
    *hne_p = 0;
    {
        DBuf dne(8, s);
        cell_rle(keys.p, kb, n, ckey.as<uint64_t>(), cstart.as<uint32_t>(), dne.as<uint32_t>(), temp.p, s);
        HDB_LAUNCH_CHECK();
        HDB_CUDA(cudaMemcpyAsync(hne_p, dne.p, 4, cudaMemcpyDeviceToHost, s));
    }
    HDB_CUDA(cudaStreamSynchronize(s));
    const uint32_t hne = *hne_p;
    g.n_nonempty = hne;
    const uint64_t nne = hne;
    // group-level arrays are sized (and scanned) by a bound on the group count instead of n:
    // a cell of c points has ceil(c / 32) <= c / 32 + 1 groups
    const uint64_t NG = std::min<uint64_t>(n, nne + n / kGroup + 1);
    keys.reset();
    tr.mark("cells+sync");
    // ---- stencil row spans per non-empty cell + query groups + hit-mask layout,
    // sized by upper bounds (groups <= NG) so that one sync reads both counts
    DBuf cspan(8 * g.nspan * nne, s), gcount(4 * (nne + 1), s), gofs(4 * (nne + 1), s);
    // the paper's dense G (Fig. 1) as a lookup, when the full grid is not much larger than the
    // data: cnext[h] = first non-empty cell with key >= h (a scan of the occupancy marks)
    DBuf cmark, cnext;
    if (nne > 0 && g.n_cells <= std::max<uint64_t>(8 * n, 1ull << 22) && g.n_cells < (1ull << 32) - 1) {
        cmark = DBuf(4 * (g.n_cells + 1), s);
        cnext = DBuf(4 * (g.n_cells + 1), s);
        DBuf ctemp(scan_temp_bytes(g.n_cells + 1), s);
        HDB_CUDA(cudaMemsetAsync(cmark.p, 0, 4 * (g.n_cells + 1), s));
        launch_cell_mark(ckey.as<uint64_t>(), nne, cmark.as<uint32_t>(), s);
        scan_u32_to_u32(cmark.as<uint32_t>(), cnext.as<uint32_t>(), g.n_cells, ctemp.p, s);
        HDB_LAUNCH_CHECK();
    }
    launch_cell_spans(ckey.as<uint64_t>(), cstart.as<uint32_t>(), nne, g.nx, g.ny, g.split, cspan.as<uint2>(),
                      gcount.as<uint32_t>(), cnext.as<uint32_t>(), s);
    cmark.reset();
    cnext.reset();
    scan_u32_to_u32(gcount.as<uint32_t>(), gofs.as<uint32_t>(), nne, temp.p, s);
    HDB_LAUNCH_CHECK();
    DBuf gstart(4 * (NG + 1), s), gcell(4 * (NG + 1), s);
    launch_group_build(cstart.as<uint32_t>(), gofs.as<uint32_t>(), nne, n, gstart.as<uint32_t>(),
                       gcell.as<uint32_t>(), s);
    HDB_LAUNCH_CHECK();
    tr.mark("spans+groups-enqueue");
    g.xy_s = xy_s.release();
    g.xp = (float4*)xp.release();
    g.counters = (unsigned int*)counters.release();
    g.ids = (uint32_t*)ids.release();
    g.ckey = (uint64_t*)ckey.release();
    g.cstart = (uint32_t*)cstart.release();
    g.cspan = (uint2*)cspan.release();
    g.gstart = (uint32_t*)gstart.release();
    g.gcell = (uint32_t*)gcell.release();
    // dense/sparse hybrid (NEXT-1): groups with few tests take the thread-per-query
    // kernel; search_kernel 3 / 4 (and the paper's kernels) keep one path for all groups.
    // The lists are built unconditionally and adopted after the final sync only if a
    // good share of the queries is sparse (no extra host sync); the mask layout keeps
    // words for every group either way.
    const int sk = ctx->opts.search_kernel;
    const uint32_t max_tests = sparse_max_tests();
    const bool classify = (sk == 0 || sk == 1 || sk == 2 || sk == 4) && max_tests > 0 && n > 0;
    // default kernel choice: small groups go to the query-lane single pass (device tables)
    const bool qrule = sk == 0 && qlanes_enabled(n, g.dtype) && (g.dtype == HDB_F32 || g.filter_b);
    DBuf dpre, spre, dl, sql, ord;
    DBuf words(4 * (NG + 1), s);   // hit-mask words per group (written with the classification)
    unsigned long long* nsp = bb + 8;
    if (classify) {
        DBuf dflag(4 * (NG + 1), s), sqn(4 * (NG + 1), s), gbin(NG + 1, s);
        uint32_t* ohist = (uint32_t*)(bb + 32);   // 2 x kOrderBins words, zeroed by the bbox init
        ord = DBuf(4 * (NG + 1), s);
        dpre = DBuf(4 * (NG + 1), s);
        spre = DBuf(4 * (NG + 1), s);
        dl = DBuf(4 * (NG + 1), s);
        sql = DBuf(8 * (n + 1), s);
        const uint32_t* ngd = gofs.as<uint32_t>() + nne;
        // nsp: [0] sparse queries, [1] candidate tests (zeroed by the bbox init)
        launch_group_class(g.cstart, g.cspan, g.nspan, g.gstart, g.gcell, ngd, NG, max_tests, qrule, dflag.as<uint32_t>(),
                           sqn.as<uint32_t>(), nsp, (uint8_t*)gbin.p, ohist, words.as<uint32_t>(), kMaskWin, s);
        launch_order_scatter((const uint8_t*)gbin.p, ngd, NG, ohist, ord.as<uint32_t>(), s);
        scan_u32_to_u32(dflag.as<uint32_t>(), dpre.as<uint32_t>(), NG, temp.p, s);
        scan_u32_to_u32(sqn.as<uint32_t>(), spre.as<uint32_t>(), NG, temp.p, s);
        launch_group_lists(g.gstart, g.gcell, ngd, NG, dpre.as<uint32_t>(), spre.as<uint32_t>(), dl.as<uint32_t>(),
                           sql.as<uint2>(), qrule, s);
        HDB_LAUNCH_CHECK();
    }
    {
        DBuf mtemp(scan_temp_bytes(NG + 1), s), moff(8 * (NG + 1), s);
        if (!classify) launch_mask_words(g, gofs.as<uint32_t>() + nne, NG, words.as<uint32_t>(), s);
        scan_u32_to_u64(words.as<uint32_t>(), moff.as<uint64_t>(), NG, mtemp.p, s);
        HDB_LAUNCH_CHECK();
        // [18] groups, [19] mask words, [20] dense groups, [21] sparse queries, [22] sparse count,
        // [23] candidate tests: gathered on the device, one pinned readback
        launch_readback(bb + 16, gofs.as<uint32_t>() + nne, moff.as<uint64_t>() + NG,
                        classify ? dpre.as<uint32_t>() + NG : nullptr, classify ? spre.as<uint32_t>() + NG : nullptr,
                        classify ? nsp : nullptr, s);
        if (g.banded)   // the band's query groups -> bb[22..23]
            launch_band_groups(g.ckey, nne, gofs.as<uint32_t>(), band_y0 * g.nx, band_y1 * g.nx, bb + 22, s);
        uint64_t* pr = dc.pin + 18;
        HDB_CUDA(cudaMemcpyAsync(pr, bb + 16, 64, cudaMemcpyDeviceToHost, s));
        HDB_CUDA(cudaEventRecord(ev1.e, s));
        tr.mark("class+order+masklayout-enqueue");
        HDB_CUDA(cudaEventSynchronize(ev1.e));
        const uint32_t hng = (uint32_t)pr[0];
        g.mask_words = pr[1];
        const uint32_t hds[2] = {(uint32_t)pr[2], (uint32_t)pr[3]};
        const uint64_t hsp = pr[4];
        g.tests_total = pr[5];
        g.n_groups = hng;
        if (g.banded) {
            g.band_g0 = pr[6];
            g.band_g1 = pr[7];
        }
        g.moff = (uint64_t*)moff.release();
        g.n_dense_groups = hng;
        g.n_sparse_q = 0;
        if (classify) g.ord = (uint32_t*)ord.release();
        // the split pays only when a good share of the queries is sparse: the thread-per-query
        // kernels run after the dense ones and a few sparse groups only add their latency
        if (classify && sk != 4 && (double)hsp >= kSparseMinShare * (double)n) {
            g.dpre = (uint32_t*)dpre.release();
            g.spre = (uint32_t*)spre.release();
            g.dl = (uint32_t*)dl.release();
            g.sql = (uint2*)sql.release();
            g.n_dense_groups = hds[0];
            g.n_sparse_q = hds[1];
            g.qsplit = qrule;
        }
    }
    g.ms_build = elapsed(ev0, ev1);
    gcount.reset();
    gofs.reset();
    temp.reset();
    misc.reset();
    tr.mark("groups+mask-layout+sync");
}

void free_dev_grid(DevGrid& g) {
    if (!g.stream) return;
    DeviceGuard dg(g.device);
    for (void* p : {(void*)g.xy_s, (void*)g.xp, (void*)g.counters, (void*)g.ids, (void*)g.ckey, (void*)g.cstart,
                    (void*)g.cspan, (void*)g.gstart, (void*)g.gcell, (void*)g.moff, (void*)g.dpre, (void*)g.spre,
                    (void*)g.dl, (void*)g.sql, (void*)g.ord})
        if (p) cudaFreeAsync(p, g.stream);   // stream-ordered: no host sync needed
    g.xy_s = nullptr;
    g.xp = nullptr;
    g.counters = nullptr;
    g.ids = g.cstart = g.gstart = g.gcell = nullptr;
    g.moff = nullptr;
    g.dpre = g.spre = g.dl = g.ord = nullptr;
    g.sql = nullptr;
    g.ckey = nullptr;
    g.cspan = nullptr;
    cudaStreamSynchronize(g.stream);
}

}  // namespace

namespace {
template <typename F>
void run_parallel(size_t k, F&& f) {
    if (k == 1) {
        f(0);
        return;
    }
    std::vector<std::exception_ptr> errs(k);
    std::vector<std::string> msgs(k);
    std::vector<std::thread> th;
    for (size_t i = 0; i < k; ++i)
        th.emplace_back([&, i] {
            try {
                f(i);
            } catch (...) {
                errs[i] = std::current_exception();
                msgs[i] = last_error();
            }
        });
    for (auto& t : th) t.join();
    for (size_t i = 0; i < k; ++i)
        if (errs[i]) {
            g_err = msgs[i];
            std::rethrow_exception(errs[i]);
        }
}

}  // namespace

// ------------------------------------------------------------------ grid
void grid_build(hdb_ctx* ctx, const void* xy, uint64_t n, hdb_dtype dt, double eps, hdb_grid** out) {
    if (dt != HDB_F64 && dt != HDB_F32) fail(HDB_EINVAL, "unknown dtype %d", (int)dt);
    if (!std::isfinite(eps) || !(eps > 0)) fail(HDB_EINVAL, "eps=%g must be finite and > 0", eps);
    if (n >= 0xffffffffull) fail(HDB_ERANGE, "n=%llu >= 2^32-1", (unsigned long long)n);
    if (n > 0 && !xy) fail(HDB_EINVAL, "xy is NULL with n=%llu", (unsigned long long)n);
    PtrInfo where = classify(xy);
    uint64_t launches0 = g_kernel_launches.load();
    auto* g = new hdb_grid;
    g->ctx = ctx;
    g->dev.resize(ctx->dev.size());
    try {
        // every device builds its copy of the grid at the same time (one host thread each)
        run_parallel(ctx->dev.size(), [&](size_t d) { build_dev(ctx, ctx->dev[d], xy, where, n, dt, eps, g->dev[d]); });
    } catch (...) {
        for (auto& dg : g->dev) free_dev_grid(dg);
        delete g;
        throw;
    }
    const DevGrid& g0 = g->dev[0];
    ctx->stats.n = n;
    ctx->stats.n_cells = g0.n_cells;
    ctx->stats.n_nonempty = g0.n_nonempty;
    ctx->stats.n_groups = g0.n_groups;
    ctx->stats.n_sparse_queries = g0.n_sparse_q;
    ctx->stats.query_lanes = g0.qsplit ? 1 : 0;
    ctx->stats.ms_grid = g0.ms_build;
    ctx->stats.kernel_launches = (uint32_t)(g_kernel_launches.load() - launches0);
    ctx->live_objects++;
    *out = g;
}

void grid_free(hdb_grid* g) {
    if (!g) return;
    for (auto& dg : g->dev) free_dev_grid(dg);
    if (g->ctx) g->ctx->live_objects--;
    delete g;
}

// ------------------------------------------------------------------ table
namespace {

struct ShardRange {
    uint64_t g0 = 0, g1 = 0;   // query groups
    uint64_t q0 = 0, q1 = 0;   // sorted query positions
};

struct ShardState {
    ShardRange r;
    DBuf cnt, off;
    DBuf masks;              // hit masks of the shard's groups (null: write pass recomputes)
    uint2* mask_base = nullptr;   // masks - moff[g0]/2, indexed by the grid-wide layout
    uint64_t pairs = 0;
    uint64_t tests = 0;
    uint64_t base = 0;   // global offset of this shard's first pair
    float ms_count = 0, ms_scan = 0, ms_write = 0;
    uint32_t write_launches = 0;
    uint64_t n_batches = 0, max_batch = 0, d2h = 0;
    uint64_t* dbeg = nullptr;   // device T by original id, written by the write kernels (null: not wanted)
    uint32_t* dcnt = nullptr;
};

// Sorted position -> group boundaries for `parts` shards balanced by the sampled counts.
std::vector<uint64_t> shard_cuts(const DevGrid& g, DevCtx& dc, const std::vector<uint32_t>& samp, uint64_t stride,
                                 uint32_t parts) {
    std::vector<uint64_t> cuts(parts + 1, 0);
    cuts[parts] = g.n_groups;
    if (parts <= 1) return cuts;
    std::vector<uint64_t> pre(samp.size() + 1, 0);
    for (size_t j = 0; j < samp.size(); ++j) pre[j + 1] = pre[j] + samp[j];
    std::vector<uint64_t> scut(parts + 1);
    hdb_balanced_cuts(pre.data(), samp.size(), parts, scut.data());
    std::vector<uint64_t> posv(parts - 1);
    for (uint32_t k = 1; k < parts; ++k) posv[k - 1] = std::min<uint64_t>(scut[k] * stride, g.n);
    cudaStream_t s = dc.main;
    DBuf dpos(8 * posv.size(), s), dgrp(8 * posv.size(), s);
    HDB_CUDA(cudaMemcpyAsync(dpos.p, posv.data(), 8 * posv.size(), cudaMemcpyHostToDevice, s));
    launch_pos_to_group(g.gstart, g.n_groups, dpos.as<uint64_t>(), (uint32_t)posv.size(), dgrp.as<uint64_t>(), s);
    std::vector<uint64_t> grp(posv.size());
    HDB_CUDA(cudaMemcpyAsync(grp.data(), dgrp.p, 8 * grp.size(), cudaMemcpyDeviceToHost, s));
    HDB_CUDA(cudaStreamSynchronize(s));
    for (uint32_t k = 1; k < parts; ++k) cuts[k] = std::max(cuts[k - 1], grp[k - 1]);
    return cuts;
}

// a6 + a7 on one device for one shard
void count_phase(hdb_ctx* ctx, DevCtx& dc, const DevGrid& g, ShardState& st) {
    ScanEpochScope scan_scope(&dc.scan_ep);
    DeviceGuard dg(dc.device);
    Trace tr("count_phase");
    cudaStream_t s = dc.main;
    const uint64_t n = g.n;
    const bool whole = st.r.g0 == 0 && st.r.g1 == g.n_groups;   // no syncs needed for the full range
    if (whole) {
        st.r.q0 = 0;
        st.r.q1 = n;
    } else if (st.r.g1 > st.r.g0) {
        uint32_t q[2] = {0, 0};
        HDB_CUDA(cudaMemcpyAsync(&q[0], g.gstart + st.r.g0, 4, cudaMemcpyDeviceToHost, s));
        HDB_CUDA(cudaMemcpyAsync(&q[1], g.gstart + st.r.g1, 4, cudaMemcpyDeviceToHost, s));
        HDB_CUDA(cudaStreamSynchronize(s));
        st.r.q0 = q[0];
        st.r.q1 = q[1];
    } else {
        st.r.q0 = st.r.q1 = 0;
    }
    st.cnt = DBuf(4 * (n ? n : 1), s);
    st.off = DBuf(8 * (n + 1), s);
    DBuf tests(8, s);
    HDB_CUDA(cudaMemsetAsync(tests.p, 0, 8, s));
    // mask table for the shard's groups (search_kernel == 2 asks for the recompute
    // write pass; an allocation failure falls back to it as well)
    if (st.r.g1 > st.r.g0 && ctx->opts.search_kernel != 2) {
        uint64_t mo[2] = {0, g.mask_words};
        if (!whole) {
            HDB_CUDA(cudaMemcpyAsync(&mo[0], g.moff + st.r.g0, 8, cudaMemcpyDeviceToHost, s));
            HDB_CUDA(cudaMemcpyAsync(&mo[1], g.moff + st.r.g1, 8, cudaMemcpyDeviceToHost, s));
            HDB_CUDA(cudaStreamSynchronize(s));
        }
        const size_t bytes = 4 * (mo[1] - mo[0]);
        void* p = nullptr;
        if (cudaMallocFromPoolAsync(&p, bytes ? bytes : 16, dc.big_pool, s) == cudaSuccess) {
            st.masks.p = p;
            st.masks.s = s;
            st.mask_base = (uint2*)p - (mo[0] >> 1);
        } else {
            cudaGetLastError();
        }
    }
    tr.mark("alloc");
    Event e0, e1, e2;
    HDB_CUDA(cudaEventRecord(e0.e, s));
    launch_count(g, st.r.g0, st.r.g1, st.cnt.as<uint32_t>(), tests.as<unsigned long long>(), ctx->opts.search_kernel,
                 0, st.mask_base, s);
    HDB_LAUNCH_CHECK();
    HDB_CUDA(cudaEventRecord(e1.e, s));
    const uint64_t len = st.r.q1 - st.r.q0;
    tr.mark("count-enqueue");
    DBuf temp(scan_temp_bytes(len + 1), s);
    scan_u32_to_u64(st.cnt.as<uint32_t>() + st.r.q0, st.off.as<uint64_t>() + st.r.q0, len, temp.p, s);
    HDB_LAUNCH_CHECK();
    HDB_CUDA(cudaEventRecord(e2.e, s));
    uint64_t* h = dc.pin + 24;   // pinned: asynchronous readbacks
    HDB_CUDA(cudaMemcpyAsync(&h[0], st.off.as<uint64_t>() + st.r.q1, 8, cudaMemcpyDeviceToHost, s));
    HDB_CUDA(cudaMemcpyAsync(&h[1], tests.p, 8, cudaMemcpyDeviceToHost, s));
    HDB_CUDA(cudaStreamSynchronize(s));
    st.pairs = h[0];
    st.tests = h[1];
    tr.mark("count+scan+sync");
    st.ms_count = elapsed(e0, e1);
    st.ms_scan = elapsed(e1, e2);
}

// Single-pass device-resident table (k_fused: count + reserve + emit per
// group; search_kernel = 4 -- measured slower than the two passes on B200,
// see DESIGN.md).  The table is sized from the sampled estimate a_b (cap = 1.25
// max(a_b, n) + 2^20 pairs).  Returns false -- nothing published, the caller
// then runs the exact two-pass path (a6-a8) -- if the mask table or the table
// cannot be allocated or a reservation passed the capacity.
bool single_pass_table(hdb_ctx* ctx, const DevGrid& g, hdb_table* t, hdb_stats& S, uint64_t est,
                       bool exact_bound = false, bool pos_space = false) {
    DevCtx& dc = ctx->dev[0];
    cudaStream_t s = dc.main;
    const uint64_t n = g.n_ids;   // rows of T (a banded grid holds fewer points)
    // est: the sampled estimate a_b (cap with headroom; a reservation past it falls back to
    // the two passes) or, exact_bound, an upper bound on P (the grid's candidate tests)
    const uint64_t cap = exact_bound ? std::max<uint64_t>(est, 1)
                                     : (uint64_t)((double)std::max<uint64_t>(est, g.n) * 1.25) + (1ull << 20);
    DBuf masks, nb;
    if (cudaMallocFromPoolAsync(&masks.p, 4 * std::max<uint64_t>(g.mask_words, 4), dc.big_pool, s) != cudaSuccess ||
        cudaMallocFromPoolAsync(&nb.p, 4 * cap, dc.big_pool, s) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    masks.s = nb.s = s;
    DBuf beg(8 * (n ? n : 1), s, dc.big_pool), cnt_id(4 * (n ? n : 1), s, dc.big_pool), scratch(32, s);
    HDB_CUDA(cudaMemsetAsync(scratch.p, 0, 32, s));
    if (g.banded) {   // a shard's table: rows outside the band stay empty
        HDB_CUDA(cudaMemsetAsync(beg.p, 0, 8 * n, s));
        HDB_CUDA(cudaMemsetAsync(cnt_id.p, 0, 4 * n, s));
    }
    unsigned long long* sc = scratch.as<unsigned long long>();
    Event e0, e1;
    HDB_CUDA(cudaEventRecord(e0.e, s));
    const uint64_t g0 = g.banded ? g.band_g0 : 0, g1 = g.banded ? g.band_g1 : g.n_groups;
    pos_space = pos_space && !g.banded && n == g.n;   // whole, unsharded tables only
    launch_fused(g, g0, g1, nullptr, sc, masks.as<uint2>(), sc + 1, cap, nb.as<uint32_t>(), beg.as<uint64_t>(),
                 cnt_id.as<uint32_t>(), (unsigned int*)(sc + 2), s, pos_space);
    if (g.dl)   // dense/sparse split: the range's sparse queries reserve on the same counter
        launch_sparse_fused(g, g0, g1, sc, sc + 1, cap, nb.as<uint32_t>(), beg.as<uint64_t>(), cnt_id.as<uint32_t>(),
                            (unsigned int*)(sc + 2), s, pos_space);
    HDB_LAUNCH_CHECK();
    HDB_CUDA(cudaEventRecord(e1.e, s));
    HDB_CUDA(cudaMemcpyAsync(dc.pin + 4, sc, 24, cudaMemcpyDeviceToHost, s));
    masks.reset();
    HDB_CUDA(cudaStreamSynchronize(s));
    const uint64_t tests = dc.pin[4], P = dc.pin[5];
    if ((uint32_t)dc.pin[6] != 0) return false;   // estimate exceeded: exact two-pass path
    t->on_device = true;
    t->device = dc.device;
    t->dstream = s;
    t->npairs = P;
    t->pos_space = pos_space;
    t->first_query = g.banded ? g.band_q0 : 0;
    t->end_query = g.banded ? g.band_q1 : n;
    if (!g.banded && n) {
        // production order of the rows (device DBSCAN walks them in this cell-sorted order)
        DBuf rw(4 * n, s, dc.big_pool);
        HDB_CUDA(cudaMemcpyAsync(rw.p, g.ids, 4 * n, cudaMemcpyDeviceToDevice, s));
        t->rows = (uint32_t*)rw.release();
    }
    t->nbrs = (uint32_t*)nb.release();
    t->begin = (uint64_t*)beg.release();
    t->count = (uint32_t*)cnt_id.release();
    S.npairs = P;
    S.candidate_tests = tests;
    S.ms_count = S.ms_scan = 0;
    S.ms_write_kernel = elapsed(e0, e1);
    S.write_launches = 1;
    S.n_batches = 1;
    S.max_batch_pairs = P;
    S.single_pass = 1;
    return true;
}

// The paper's kernels (search_kernel 7 / 8; NEXT-3): GPUCalcGlobal (Alg. 2) or
// GPUCalcShared (Alg. 3) append the key/value result set R with atomics into a
// buffer sized from the sampled estimate ((1 + 2 alpha) a_b + n, P:736-741,
// P:812-823); the append counter keeps counting past the capacity, so an
// overflow reruns the kernel once at the exact |R| (reading R14).  R is then
// sorted by key (Alg. 4 line 7, the paper's sort_by_key; here the library's
// LSD radix sort) and T's ranges are read off the sorted keys
// (ConstructNeighborTable).  Device-resident whole tables only.
void paper_table(hdb_ctx* ctx, const DevGrid& g, hdb_table* t, hdb_stats& S, uint64_t est, int which) {
    DevCtx& dc = ctx->dev[0];
    cudaStream_t s = dc.main;
    const uint64_t n = g.n;
    uint64_t cap = (uint64_t)((1.0 + 2.0 * ctx->opts.alpha) * (double)est) + n + 1024;
    DBuf ctr(8, s);
    float ms_search = 0;
    uint64_t P = 0;
    DBuf rkey, rval;
    for (int attempt = 0; attempt < 2; ++attempt) {
        if (cap >= (1ull << 32)) cap = (1ull << 32) - 1;
        rkey = DBuf(4 * cap, s);
        rval = DBuf(4 * cap, s);
        HDB_CUDA(cudaMemsetAsync(ctr.p, 0, 8, s));
        Event e0, e1;
        HDB_CUDA(cudaEventRecord(e0.e, s));
        launch_paper_search(g, which, ctr.as<unsigned long long>(), cap, rkey.as<uint32_t>(), rval.as<uint32_t>(), s);
        HDB_LAUNCH_CHECK();
        HDB_CUDA(cudaEventRecord(e1.e, s));
        HDB_CUDA(cudaMemcpyAsync(dc.pin + 4, ctr.p, 8, cudaMemcpyDeviceToHost, s));
        HDB_CUDA(cudaStreamSynchronize(s));
        ms_search += elapsed(e0, e1);
        P = dc.pin[4];
        if (P <= cap) break;
        ++S.pool_grows;
        cap = P;   // exact |R| now known
        if (P >= (1ull << 32) - 1)
            fail(HDB_ERANGE, "the paper kernels' result set (%llu pairs) needs 32-bit positions",
                 (unsigned long long)P);
    }
    // Alg. 4 line 7: sort R by key (stable LSD radix sort on the key's bits)
    int bits = 1;
    while (bits < 32 && (1ull << bits) < n) ++bits;
    DBuf k1(4 * (P ? P : 1), s), v1(4 * (P ? P : 1), s), tmp(radix_sort_temp_bytes(P ? P : 1), s);
    DBuf beg(8 * (n ? n : 1), s), cnt(4 * (n ? n : 1), s);
    Event e2, e3;
    HDB_CUDA(cudaEventRecord(e2.e, s));
    const int where = radix_sort_pairs(rkey.p, rval.as<uint32_t>(), k1.p, v1.as<uint32_t>(), 4, P, bits, tmp.p, s);
    const uint32_t* ks = where ? k1.as<uint32_t>() : rkey.as<uint32_t>();
    launch_rows_from_keys(ks, P, n, beg.as<uint64_t>(), cnt.as<uint32_t>(), s);
    HDB_LAUNCH_CHECK();
    HDB_CUDA(cudaEventRecord(e3.e, s));
    HDB_CUDA(cudaStreamSynchronize(s));
    t->on_device = true;
    t->device = dc.device;
    t->dstream = s;
    t->npairs = P;
    t->first_query = 0;
    t->end_query = n;
    t->nbrs = (uint32_t*)(where ? v1.release() : rval.release());
    t->begin = (uint64_t*)beg.release();
    t->count = (uint32_t*)cnt.release();
    S.npairs = P;
    S.candidate_tests = 0;
    S.ms_count = S.ms_scan = 0;
    S.ms_write_kernel = ms_search;
    S.ms_sort = elapsed(e2, e3);
    S.write_launches = 1;
    S.n_batches = 1;
    S.max_batch_pairs = P;
}

void ensure_batch_buf(DevCtx& dc, size_t si, size_t pairs, uint64_t* grows) {
    if (dc.batch_buf.size() <= si) {
        dc.batch_buf.resize(si + 1, nullptr);
        dc.batch_cap.resize(si + 1, 0);
    }
    if (dc.batch_cap[si] >= pairs && dc.batch_buf[si]) return;
    if (dc.batch_buf[si]) {
        HDB_CUDA(cudaStreamSynchronize(dc.streams[si]));
        cudaFree(dc.batch_buf[si]);
        dc.batch_buf[si] = nullptr;
        dc.batch_cap[si] = 0;
    }
    size_t cap = std::max<size_t>(pairs, 1024);
    cap += cap / 8;
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, cap * 4);
    if (e != cudaSuccess) {
        cudaGetLastError();
        fail(HDB_ENOMEM, "device batch buffer of %zu pairs: %s", cap, cudaGetErrorString(e));
    }
    dc.batch_buf[si] = (uint32_t*)p;
    dc.batch_cap[si] = cap;
    ++*grows;
}

// a8 + a9 for one shard: batches cut on exact counts, round-robin on streams,
// each batch written into a per-stream device buffer and DMA'd into the host
// table at its final offset.
void write_phase_host(hdb_ctx* ctx, DevCtx& dc, const DevGrid& g, ShardState& st, uint32_t* h_nbrs,
                      uint64_t batch_pairs, uint64_t* grows) {
    DeviceGuard dg(dc.device);
    if (st.pairs == 0) return;
    cudaStream_t s = dc.main;
    const uint32_t S = (uint32_t)dc.streams.size();
    uint64_t nb = (st.pairs + batch_pairs - 1) / batch_pairs;
    nb = std::max<uint64_t>(nb, 1);
    nb = std::min<uint64_t>(nb, std::max<uint64_t>(1, st.r.g1 - st.r.g0));
    DBuf dcut(8 * (nb + 1) * 2, s);
    uint64_t* gcut = dcut.as<uint64_t>();
    uint64_t* pcut = gcut + (nb + 1);
    // offsets are relative to the shard start: off[q0] == 0
    launch_batch_cuts(g.gstart, st.off.as<uint64_t>(), st.r.g0, st.r.g1, (uint32_t)nb, gcut, pcut, s);
    HDB_LAUNCH_CHECK();
    std::vector<uint64_t> hc(2 * (nb + 1));
    HDB_CUDA(cudaMemcpyAsync(hc.data(), dcut.p, 8 * hc.size(), cudaMemcpyDeviceToHost, s));
    HDB_CUDA(cudaStreamSynchronize(s));
    const uint64_t* hg = hc.data();
    const uint64_t* hp = hc.data() + (nb + 1);
    uint64_t maxb = 0;
    for (uint64_t b = 0; b < nb; ++b) maxb = std::max(maxb, hp[b + 1] - hp[b]);
    for (uint32_t i = 0; i < S && i < nb; ++i) ensure_batch_buf(dc, i, maxb, grows);
    Event ready;
    HDB_CUDA(cudaEventRecord(ready.e, s));
    std::vector<Event> evs(2 * nb);
    const bool tl = timeline_on();
    std::vector<Event> cev(tl ? nb : 0);   // end of each batch's D2H copy (timeline only)
    for (uint64_t b = 0; b < nb; ++b) {
        const uint32_t si = (uint32_t)(b % S);
        cudaStream_t ss = dc.streams[si];
        const uint64_t pairs_b = hp[b + 1] - hp[b];
        if (b < S) HDB_CUDA(cudaStreamWaitEvent(ss, ready.e, 0));
        HDB_CUDA(cudaEventRecord(evs[2 * b].e, ss));
        launch_write(g, hg[b], hg[b + 1], st.off.as<uint64_t>(), hp[b], dc.batch_buf[si], ctx->opts.search_kernel,
                     1 + (int)si, st.mask_base, ss, st.dbeg, st.dcnt);
        HDB_LAUNCH_CHECK();
        HDB_CUDA(cudaEventRecord(evs[2 * b + 1].e, ss));
        if (pairs_b)
            HDB_CUDA(cudaMemcpyAsync(h_nbrs + st.base + hp[b], dc.batch_buf[si], 4 * pairs_b, cudaMemcpyDeviceToHost,
                                     ss));
        if (tl) HDB_CUDA(cudaEventRecord(cev[b].e, ss));
        st.d2h += 4 * pairs_b;
    }
    for (uint32_t i = 0; i < S; ++i) HDB_CUDA(cudaStreamSynchronize(dc.streams[i]));
    for (uint64_t b = 0; b < nb; ++b) st.ms_write += elapsed(evs[2 * b], evs[2 * b + 1]);
    if (tl) {
        std::string js = "{\"timeline\": \"host_table_write\", \"device\": " + std::to_string(dc.device) +
                         ", \"batches\": [";
        for (uint64_t b = 0; b < nb; ++b) {
            char buf[256];
            snprintf(buf, sizeof buf,
                     "%s{\"b\": %llu, \"stream\": %u, \"pairs\": %llu, \"write\": [%.4f, %.4f], \"d2h\": [%.4f, %.4f]}",
                     b ? ", " : "", (unsigned long long)b, (unsigned)(b % S), (unsigned long long)(hp[b + 1] - hp[b]),
                     elapsed(evs[0], evs[2 * b]), elapsed(evs[0], evs[2 * b + 1]), elapsed(evs[0], evs[2 * b + 1]),
                     elapsed(evs[0], cev[b]));
            js += buf;
        }
        js += "]}";
        fprintf(stderr, "%s\n", js.c_str());
    }
    st.write_launches += (uint32_t)nb;
    st.n_batches = nb;
    st.max_batch = maxb;
}

template <typename T>
T* pool_get(hdb_table* t, size_t count, size_t* cap) {
    return (T*)t->pool->acquire(count * sizeof(T), cap);
}

}  // namespace

// DBSCAN on a device-resident table (NEXT-4): labels / core may be host or
// device pointers (core may be null); returns the number of clusters.
uint32_t dbscan_device(const hdb_table* t, uint32_t minpts, int32_t* labels, uint8_t* core) {
    DeviceGuard dg(t->device);
    cudaStream_t s = t->dstream;
    const uint64_t n = t->n;
    if (n == 0) return 0;
    const PtrInfo li = classify(labels), ci = classify(core);
    const bool lab_dev = li.loc == Loc::Device && li.device == t->device;
    const bool core_dev = core && ci.loc == Loc::Device && ci.device == t->device;
    DBuf dlab, dcore(n, s), parent(4 * n, s), root(4 * n, s), is_root(4 * n, s), rank(4 * (n + 1), s),
        temp(scan_temp_bytes(n + 1), s), giant(16, s), bits(8 * ((n + 31) / 32), s), sched(8 * 1024, s), pre(8 * (n + 1), s);
    int32_t* L = labels;
    if (!lab_dev) {
        dlab = DBuf(4 * n, s);
        L = dlab.as<int32_t>();
    }
    // id space: the core flags are computed in the caller's array (or a device copy of it);
    // position space: by position in dcore, then written out by id (into core / its copy)
    DBuf ccopy;
    uint8_t* C = (core_dev && !t->pos_space) ? core : dcore.as<uint8_t>();
    uint8_t* Cout = nullptr;
    if (t->pos_space && core) {
        if (core_dev) {
            Cout = core;
        } else {
            ccopy = DBuf(n, s);
            Cout = ccopy.as<uint8_t>();
        }
    }
    launch_dbscan_device(t->begin, t->count, t->nbrs, t->rows, n, t->npairs, minpts, C, parent.as<uint32_t>(),
                         root.as<uint32_t>(), is_root.as<uint32_t>(), rank.as<uint32_t>(), giant.as<uint32_t>(),
                         bits.as<uint32_t>(), sched.as<uint32_t>(), pre.as<uint64_t>(), temp.p, L, s, t->pos_space,
                         Cout);
    if (t->pos_space) C = Cout;   // the by-id flags (null when not asked for)
    HDB_LAUNCH_CHECK();
    uint32_t k = 0;
    HDB_CUDA(cudaMemcpyAsync(&k, rank.as<uint32_t>() + n, 4, cudaMemcpyDeviceToHost, s));
    if (!lab_dev) HDB_CUDA(cudaMemcpyAsync(labels, L, 4 * n, cudaMemcpyDeviceToHost, s));
    if (core && !core_dev) HDB_CUDA(cudaMemcpyAsync(core, C, n, cudaMemcpyDeviceToHost, s));   // (by id)
    HDB_CUDA(cudaStreamSynchronize(s));
    return k;
}

void table_free(hdb_table* t) {
    if (!t) return;
    if (t->on_device) {
        DeviceGuard dg(t->device);
        for (void* p : {(void*)t->begin, (void*)t->count, (void*)t->nbrs, (void*)t->rows})
            if (p) cudaFreeAsync(p, t->dstream);   // stream-ordered: no host sync needed
    } else if (t->pool) {
        t->pool->release(t->begin, t->cap_begin);
        t->pool->release(t->count, t->cap_count);
        t->pool->release(t->nbrs, t->cap_nbrs);
    } else if (t->malloced) {
        free(t->begin);
        free(t->count);
        free(t->nbrs);
    }
    if (t->ctx) t->ctx->live_objects--;
    delete t;
}

// The grid as the count -> scan -> write paths see it: a query-lane split (the small
// groups of k_qlanes) is a device-single-pass-only classification, so those paths run
// every group through the warp-per-group kernels (as without a split).
DevGrid without_qsplit(const DevGrid& g) {
    DevGrid r = g;
    if (r.qsplit) {
        r.qsplit = false;
        r.dl = r.dpre = r.spre = nullptr;
        r.sql = nullptr;
        r.n_sparse_q = 0;
        r.n_dense_groups = r.n_groups;
    }
    return r;
}

void neighbor_table(hdb_ctx* ctx, const hdb_grid* grid, bool device_resident, hdb_table** out, bool pos_space) {
    auto t_wall0 = std::chrono::steady_clock::now();
    const uint64_t launches0 = g_kernel_launches.load();
    hdb_stats& S = ctx->stats;
    const DevGrid& G0 = grid->dev[0];
    const uint64_t n = G0.n_ids;    // rows of T
    const uint64_t n_pts = G0.n;    // points of the grid (a process shard's band: fewer)
    const bool banded = G0.banded;
    S.n = n;
    S.n_cells = G0.n_cells;
    S.n_nonempty = G0.n_nonempty;
    S.n_groups = G0.n_groups;
    S.n_sparse_queries = G0.n_sparse_q;
    S.query_lanes = G0.qsplit ? 1 : 0;
    S.bytes_d2h = 0;
    S.pool_grows = 0;
    S.n_streams = ctx->opts.n_streams;
    const uint32_t R_proc = ctx->opts.shard_count > 0 ? (uint32_t)ctx->opts.shard_count : 1;
    const uint32_t rank = ctx->opts.shard_count > 0 ? (uint32_t)ctx->opts.shard_rank : 0;
    const size_t ndev = device_resident ? 1 : grid->dev.size();
    S.n_devices = (int)ndev;
    std::vector<DevGrid> gx;   // the grids of the two-pass paths (no query-lane split)
    for (const DevGrid& d : grid->dev) gx.push_back(without_qsplit(d));

    auto* t = new hdb_table;
    t->n = n;
    t->eps = G0.eps;
    t->dtype = G0.dtype;
    t->host_threads = ctx->opts.host_threads;
    std::vector<ShardState> sh(ndev);
    try {
        Trace tr("neighbor_table");
        DevCtx& dc0 = ctx->dev[0];
        DeviceGuard dg0(dc0.device);
        // a banded grid (process shard) is already this rank's part: no further cuts
        const uint32_t parts = banded ? 1u : R_proc * (uint32_t)ndev;
        // ---- dense device-resident whole table: the single pass sized by the exact upper
        // bound P <= candidate tests (known from the grid), no sampled estimate needed (the
        // sample kernel and its readback sync were ~3% of a C2 step)
        // (with the dense/sparse split: k_fused on the dense groups + the thread-per-query
        // single pass on the sparse queries, whatever the pairs per query)
        if (device_resident && parts == 1 && ctx->opts.search_kernel == 0 && n_pts > 0 &&
            (G0.dl || G0.tests_total >= (uint64_t)(kFusedDirectTestsPerQuery * (double)n_pts)) &&
            4.0 * (double)G0.tests_total <= kFusedDirectMemShare * (double)dc0.total_mem) {
            S.sample_size = 0;
            S.sample_pairs = 0;
            S.est_pairs = 0;
            S.ms_sample = 0;
            S.ms_sort = 0;
            S.planned_batch_pairs = S.planned_batches = 0;
            if (single_pass_table(ctx, G0, t, S, G0.tests_total, true, pos_space)) {   // (cannot overflow)
                tr.mark("single-pass (exact bound)");
                S.kernel_launches = (uint32_t)(g_kernel_launches.load() - launches0);
                S.ms_table_wall =
                    std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_wall0).count();
                t->ctx = ctx;
                ctx->live_objects++;
                *out = t;
                return;
            }
        }
        // ---- a5: sampled count + plan (device 0)
        const double f = ctx->opts.sample_fraction;
        const uint64_t stride = std::max<uint64_t>(1, (uint64_t)std::floor(1.0 / f));
        const uint64_t ns = n_pts ? (n_pts + stride - 1) / stride : 0;
        std::vector<uint32_t> samp;
        cudaStream_t s0 = dc0.main;
        DBuf dsamp(4 * (ns ? ns : 1), s0), dsum(8, s0);
        Event es0, es1;
        HDB_CUDA(cudaMemsetAsync(dsum.p, 0, 8, s0));
        HDB_CUDA(cudaEventRecord(es0.e, s0));
        launch_sample_count(gx[0], stride, ns, dsamp.as<uint32_t>(), dsum.as<unsigned long long>(), s0);
        HDB_LAUNCH_CHECK();
        HDB_CUDA(cudaEventRecord(es1.e, s0));
        // e_b lands in pinned scratch; unsharded calls read it after the count pass's sync
        HDB_CUDA(cudaMemcpyAsync(dc0.pin, dsum.p, 8, cudaMemcpyDeviceToHost, s0));
        if (parts > 1 && ns) {   // shard cuts need the per-sample counts now
            samp.resize(ns);
            HDB_CUDA(cudaMemcpyAsync(samp.data(), dsamp.p, 4 * ns, cudaMemcpyDeviceToHost, s0));
            HDB_CUDA(cudaStreamSynchronize(s0));
        }
        // ---- query shards: processes x devices, balanced by sampled counts
        if (banded) {
            sh[0].r.g0 = G0.band_g0;
            sh[0].r.g1 = G0.band_g1;
        } else {
            std::vector<uint64_t> cuts = shard_cuts(gx[0], dc0, samp, stride, parts);
            for (size_t d = 0; d < ndev; ++d) {
                const uint32_t k = rank * (uint32_t)ndev + (uint32_t)d;
                sh[d].r.g0 = cuts[k];
                sh[d].r.g1 = cuts[k + 1];
            }
        }
        tr.mark("sample+cuts");
        S.single_pass = 0;
        S.ms_sort = 0;
        bool single = false;
        const int sk = ctx->opts.search_kernel;
        if ((sk == kPaperGlobal || sk == kPaperShared) && !(device_resident && parts == 1 && !banded))
            fail(HDB_EINVAL, "search_kernel %d (the paper's kernels) builds device-resident, unsharded tables only", sk);
        if ((sk == kPaperGlobal || sk == kPaperShared) && n > 0) {
            HDB_CUDA(cudaStreamSynchronize(s0));   // e_b is in dc0.pin[0]
            const uint64_t eb = dc0.pin[0];
            S.sample_size = ns;
            S.sample_pairs = eb;
            S.est_pairs = eb * stride;
            S.ms_sample = elapsed(es0, es1);
            paper_table(ctx, G0, t, S, eb * stride, sk);
            single = true;
            tr.mark("paper-kernel");
        }
        // single pass (k_fused): asked for (search_kernel 4) or chosen for dense tables;
        // the dense/sparse split keeps the two passes (the sparse queries' kernels
        // write at scanned offsets)
        if (!single && device_resident && parts == 1 && (sk == 4 || sk == 0) && n_pts > 0) {
            HDB_CUDA(cudaStreamSynchronize(s0));   // e_b is in dc0.pin[0]
            const uint64_t eb = dc0.pin[0];
            const bool fused = sk == 4 || (double)(eb * stride) >= kFusedMinPairsPerQuery * (double)n_pts;
            if (fused) {
                S.sample_size = ns;
                S.sample_pairs = eb;
                S.est_pairs = eb * stride;
                S.ms_sample = elapsed(es0, es1);
                single = single_pass_table(ctx, G0, t, S, eb * stride, false, pos_space);
            }
            if (single) {
                double bb = 0;
                uint64_t nbp = 0;
                hdb_plan_batches((double)S.est_pairs, ctx->opts.alpha, ctx->opts.n_streams, &bb, &nbp);
                S.planned_batch_pairs = (uint64_t)std::ceil(bb);
                S.planned_batches = nbp;
            }
            tr.mark("single-pass");
        }
        if (!single) {
            // ---- a6/a7 on every device
            run_parallel(ndev, [&](size_t d) { count_phase(ctx, ctx->dev[d], gx[d], sh[d]); });
            tr.mark("count_phase");
            HDB_CUDA(cudaStreamSynchronize(s0));   // no-op when device 0 ran the count pass (same stream)
            {
                const uint64_t eb = dc0.pin[0];
                S.sample_size = ns;
                S.sample_pairs = eb;
                S.est_pairs = eb * stride;   // a_b = e_b / f  (reading R15)
                S.ms_sample = elapsed(es0, es1);
            }
            double bb_plan = 0;
            uint64_t nb_plan = 0;
            hdb_plan_batches((double)S.est_pairs, ctx->opts.alpha, ctx->opts.n_streams, &bb_plan, &nb_plan);
            uint64_t batch_pairs = ctx->opts.batch_pairs ? ctx->opts.batch_pairs : (uint64_t)std::ceil(bb_plan);
            batch_pairs = std::max<uint64_t>(batch_pairs, 1);
            S.planned_batch_pairs = batch_pairs;
            S.planned_batches = ctx->opts.batch_pairs
                                    ? (uint64_t)std::ceil((1.0 + ctx->opts.alpha) * (double)S.est_pairs / (double)batch_pairs)
                                    : nb_plan;
            // ---- the final gather of counts: shard bases
            uint64_t P = 0;
            for (size_t d = 0; d < ndev; ++d) {
                sh[d].base = P;
                P += sh[d].pairs;
            }
            S.npairs = P;
            S.candidate_tests = 0;
            S.ms_count = S.ms_scan = 0;
            for (auto& st : sh) {
                S.candidate_tests += st.tests;
                S.ms_count = std::max(S.ms_count, (double)st.ms_count);
                S.ms_scan = std::max(S.ms_scan, (double)st.ms_scan);
            }
            if (ctx->opts.host_budget_bytes && 4 * P > ctx->opts.host_budget_bytes && !device_resident)
                fail(HDB_ENOMEM, "table needs %llu bytes (P=%llu) > host budget %llu", (unsigned long long)(4 * P),
                     (unsigned long long)P, (unsigned long long)ctx->opts.host_budget_bytes);
            t->npairs = P;
            const bool whole = (parts == 1) && !banded;
            // this process's rows: [first_query, end_query) of the sorted order -- the whole
            // table unless the process is one of several shards (R_proc > 1); empty shards
            // (q0 = q1 = 0) do not count; a band knows its global range
            if (banded) {
                t->first_query = G0.band_q0;
                t->end_query = G0.band_q1;
            } else if (R_proc == 1) {
                t->first_query = 0;
                t->end_query = n;
            } else {
                t->first_query = t->end_query = 0;
                bool any = false;
                for (size_t d = 0; d < ndev; ++d) {
                    if (sh[d].r.q1 <= sh[d].r.q0) continue;
                    t->first_query = any ? std::min(t->first_query, sh[d].r.q0) : sh[d].r.q0;
                    t->end_query = any ? std::max(t->end_query, sh[d].r.q1) : sh[d].r.q1;
                    any = true;
                }
            }

            if (device_resident) {
                // ---- a8 into a device-resident table
                DevCtx& dc = ctx->dev[0];
                const DevGrid& g = gx[0];
                ShardState& st = sh[0];
                cudaStream_t s = dc.main;
                t->on_device = true;
                t->device = dc.device;
                t->dstream = s;
                DBuf nb(4 * (P ? P : 1), s, dc.big_pool), beg(8 * (n ? n : 1), s, dc.big_pool),
                    cnt(4 * (n ? n : 1), s, dc.big_pool);
                if (!whole) {
                    HDB_CUDA(cudaMemsetAsync(beg.p, 0, 8 * (n ? n : 1), s));
                    HDB_CUDA(cudaMemsetAsync(cnt.p, 0, 4 * (n ? n : 1), s));
                }
                Event e0, e1;
                HDB_CUDA(cudaEventRecord(e0.e, s));
                // the write kernels also write T by original id (begin/count) for their rows
                launch_write(g, st.r.g0, st.r.g1, st.off.as<uint64_t>(), 0, nb.as<uint32_t>(), ctx->opts.search_kernel, 1,
                             st.mask_base, s, beg.as<uint64_t>(), cnt.as<uint32_t>());
                HDB_LAUNCH_CHECK();
                HDB_CUDA(cudaEventRecord(e1.e, s));
                HDB_CUDA(cudaStreamSynchronize(s));
                st.ms_write = elapsed(e0, e1);
                tr.mark("alloc+write+scatter+sync");
                st.write_launches = 1;
                st.n_batches = 1;
                st.max_batch = P;
                if (whole && n) {
                    // production order of the rows: DBSCAN walks them in this (cell-sorted) order so
                    // that consecutive rows share neighbours (cache locality of the union-find)
                    DBuf rw(4 * n, s);
                    HDB_CUDA(cudaMemcpyAsync(rw.p, g.ids, 4 * n, cudaMemcpyDeviceToDevice, s));
                    t->rows = (uint32_t*)rw.release();
                }
                t->nbrs = (uint32_t*)nb.release();
                t->begin = (uint64_t*)beg.release();
                t->count = (uint32_t*)cnt.release();
            } else {
                // ---- a8/a9/a10 into the host table
                t->pool = ctx->pinned;
                uint64_t grows0 = ctx->pinned->grows;
                t->nbrs = pool_get<uint32_t>(t, P ? P : 1, &t->cap_nbrs);
                t->begin = pool_get<uint64_t>(t, n ? n : 1, &t->cap_begin);
                t->count = pool_get<uint32_t>(t, n ? n : 1, &t->cap_count);
                if (!whole) {
                    memset(t->begin, 0, 8 * (n ? n : 1));
                    memset(t->count, 0, 4 * (n ? n : 1));
                }
                tr.mark("pinned-pool");
                // begin/count by original id: written on the device by the write kernels
                // (one device, whole range), then one copy each
                DBuf beg, cnt;
                if (whole) {
                    DevCtx& dc = ctx->dev[0];
                    DeviceGuard dg(dc.device);
                    beg = DBuf(8 * (n ? n : 1), dc.main);
                    cnt = DBuf(4 * (n ? n : 1), dc.main);
                    sh[0].dbeg = beg.as<uint64_t>();
                    sh[0].dcnt = cnt.as<uint32_t>();
                }
                std::vector<uint64_t> dev_grows(ndev, 0);
                run_parallel(ndev, [&](size_t d) {
                    write_phase_host(ctx, ctx->dev[d], gx[d], sh[d], t->nbrs, batch_pairs, &dev_grows[d]);
                });
                tr.mark("write+d2h");
                if (whole) {
                    DevCtx& dc = ctx->dev[0];
                    DeviceGuard dg(dc.device);
                    cudaStream_t s = dc.main;
                    if (n) {
                        HDB_CUDA(cudaMemcpyAsync(t->begin, beg.p, 8 * n, cudaMemcpyDeviceToHost, s));
                        HDB_CUDA(cudaMemcpyAsync(t->count, cnt.p, 4 * n, cudaMemcpyDeviceToHost, s));
                    }
                    HDB_CUDA(cudaStreamSynchronize(s));
                    S.bytes_d2h += 12 * n;
                } else {
                    run_parallel(ndev, [&](size_t d) {
                        ShardState& st = sh[d];
                        const uint64_t len = st.r.q1 - st.r.q0;
                        if (!len) return;
                        DeviceGuard dg(ctx->dev[d].device);
                        cudaStream_t s = ctx->dev[d].main;
                        std::vector<uint32_t> ids(len), cnt(len);
                        std::vector<uint64_t> off(len);
                        HDB_CUDA(cudaMemcpyAsync(ids.data(), grid->dev[d].ids + st.r.q0, 4 * len, cudaMemcpyDeviceToHost, s));
                        HDB_CUDA(cudaMemcpyAsync(cnt.data(), st.cnt.as<uint32_t>() + st.r.q0, 4 * len,
                                                 cudaMemcpyDeviceToHost, s));
                        HDB_CUDA(cudaMemcpyAsync(off.data(), st.off.as<uint64_t>() + st.r.q0, 8 * len,
                                                 cudaMemcpyDeviceToHost, s));
                        HDB_CUDA(cudaStreamSynchronize(s));
                        for (uint64_t i = 0; i < len; ++i) {
                            t->begin[ids[i]] = off[i] + st.base;
                            t->count[ids[i]] = cnt[i];
                        }
                        st.d2h += 16 * len;
                    });
                }
                for (size_t d = 0; d < ndev; ++d) S.pool_grows += dev_grows[d];
                S.pool_grows += ctx->pinned->grows - grows0;
                if (ctx->opts.sort_lists) {
                    const int T = resolve_threads(ctx->opts.host_threads);
                    run_parallel((size_t)T, [&](size_t k) {
                        for (uint64_t p = k; p < n; p += (uint64_t)T)
                            std::sort(t->nbrs + t->begin[p], t->nbrs + t->begin[p] + t->count[p]);
                    });
                }
            }
            S.n_batches = S.max_batch_pairs = 0;
            S.ms_write_kernel = 0;
            S.write_launches = 0;
            for (auto& st : sh) {
                S.n_batches += st.n_batches;
                S.max_batch_pairs = std::max(S.max_batch_pairs, st.max_batch);
                S.ms_write_kernel += st.ms_write;
                S.write_launches += st.write_launches;
                S.bytes_d2h += st.d2h;
            }
        }
    } catch (...) {
        for (auto& st : sh) {
            st.cnt.reset();
            st.off.reset();
            st.masks.reset();
        }
        table_free(t);
        throw;
    }
    for (size_t d = 0; d < ndev; ++d) {
        DeviceGuard dg(ctx->dev[d].device);
        sh[d].cnt.reset();
        sh[d].off.reset();
        sh[d].masks.reset();
    }
    S.kernel_launches = (uint32_t)(g_kernel_launches.load() - launches0);
    S.ms_table_wall =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_wall0).count();
    t->ctx = ctx;
    ctx->live_objects++;
    *out = t;
}

}  // namespace hdb
