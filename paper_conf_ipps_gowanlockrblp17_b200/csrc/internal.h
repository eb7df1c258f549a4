// internal.h -- shared declarations of libhdb (kernels + host orchestration).
// Not part of the public ABI (include/hdb.h is).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "hdb.h"

namespace hdb {

// ---------------------------------------------------------------- errors
extern std::atomic<uint64_t> g_kernel_launches;   // kernels launched by this process
void set_error(const char* fmt, ...);
struct Error {
    hdb_status st;
};
[[noreturn]] void fail(hdb_status st, const char* fmt, ...);
#define HDB_CUDA(call)                                                                      \
    do {                                                                                    \
        cudaError_t e_ = (call);                                                            \
        if (e_ != cudaSuccess)                                                              \
            ::hdb::fail(e_ == cudaErrorMemoryAllocation ? HDB_ENOMEM : HDB_ECUDA,           \
                        "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__,   \
                        __LINE__);                                                          \
    } while (0)
#define HDB_LAUNCH_CHECK() HDB_CUDA(cudaGetLastError())

// Warps per search CTA and queries per group (one warp's query tile).
constexpr int kGroup = 32;
constexpr int kSearchThreads = 256;
constexpr int kCounterSlots = 64;   // slot 0: count pass; 1 + stream index: write passes
constexpr int kMaxCellSplit = 6;    // cell_split k <= 6: 2k+1 <= 13 stencil row spans (kMaxSpans)
// Query-lane blocks (k_qlanes): a group is SMALL -- its queries
// take one lane each -- when its hit words fit (sum over the stencil rows of
// ceil((len/2 + 1) / 16) <= kQW) and every row span holds <= kQS candidates; a block's
// queries lie in one cell row at most kQCX columns apart (bounds the block-local filter).
constexpr int kQW = 8;
constexpr int kQS = 256;
constexpr int kQCX = 24;

// ---------------------------------------------------------------- grid
// One device's copy of the grid (Fig. 1 re-laid out):
// points sorted by cell key h = cy*nx + cx; only NON-EMPTY cells are stored
// (key, start), so sparse extents cost nothing; every non-empty cell carries
// its three stencil row spans (contiguous ranges of sorted positions).
struct DevGrid {
    int device = 0;
    hdb_dtype dtype = HDB_F64;
    uint64_t n = 0;                // points of this grid
    uint64_t n_ids = 0;            // the id space (rows of T): the input's point count
    // process-shard band: the grid holds the cell rows of shard r plus k halo
    // rows; its queries are the groups [band_g0, band_g1), rows [band_q0, band_q1) of the
    // GLOBAL cell-sorted order; ids are input rows
    bool banded = false;
    uint64_t band_g0 = 0, band_g1 = 0, band_q0 = 0, band_q1 = 0;
    double eps = 0, w = 0, inv_w = 0;
    double e2_d = 0;     // fl(eps*eps) in f64
    float e2_f = 0;      // fl(eps_f*eps_f) in f32 (f32 mode) / fl32(e2_d) (f64 filter)
    float band = 0;      // f64 mode, bbox-centre filter: |t| <= band => decide in exact f64
    bool filter = false; // f64 mode: bbox-centre filter usable (recompute write variant)
    float band_l = 0;    // f64 mode, group-local filter (count pass)
    float nb2_l = 0;     //   -(band_l (1 + 2^-20))^2, rounded away from zero
    bool filter_l = false;
    float nb2_b = 0;     // f64 mode, query-lane block filter (origin: the block's first query)
    bool filter_b = false;
    double xmin = 0, ymin = 0, xmax = 0, ymax = 0;
    double ox = 0, oy = 0;  // f64 mode: origin of the f32 filter coordinates
    uint32_t nx = 1, ny = 1;
    uint32_t split = 1;            // k: cell width eps/k, stencil (2k+1) x (2k+1) cells
    uint32_t nspan = 3;            // 2k+1 row spans per non-empty cell
    uint64_t n_cells = 0, n_nonempty = 0, n_groups = 0;
    void* xy_s = nullptr;          // [n] double2 / float2, cell order (exact coordinates)
    float4* xp = nullptr;          // [n/2+1] paired-SoA f32 coords {x_2k, x_2k+1, y_2k, y_2k+1}: the
                                   // filter coords x-ox, y-oy (f64 mode) / the exact coords (f32 mode)
    unsigned int* counters = nullptr;  // [kCounterSlots] work counters of the search kernels
    uint32_t* ids = nullptr;       // [n] sorted pos -> original id  (A)
    uint64_t* ckey = nullptr;      // [n_nonempty] cell key of each non-empty cell (ascending)
    uint32_t* cstart = nullptr;    // [n_nonempty+1] first sorted pos of each non-empty cell (G)
    uint2* cspan = nullptr;        // [nspan*n_nonempty] stencil row spans [lo,hi) per non-empty cell
    uint32_t* gstart = nullptr;    // [n_groups+1] first sorted pos of each query group
    uint32_t* gcell = nullptr;     // [n_groups] non-empty cell index of each query group
    uint64_t* moff = nullptr;      // [n_groups+1] first 32-bit word of each group's hit masks
    uint64_t mask_words = 0;       // moff[n_groups]
    // dense/sparse hybrid (NEXT-1): null when every group takes the warp-per-group path
    uint32_t* dpre = nullptr;      // [n_groups+1] dense groups before g
    uint32_t* dl = nullptr;        // [#dense] the dense groups, ascending
    uint32_t* ord = nullptr;       // [n_groups] cost order: dense groups heaviest first, then the sparse
                                   // ones (whole-range count / write launches visit groups in this order)
    uint32_t* spre = nullptr;      // [n_groups+1] sparse queries before group g
    uint2* sql = nullptr;          // [n_sparse_q] {sorted position, non-empty cell} of each sparse query
    uint64_t n_sparse_q = 0, n_dense_groups = 0;
    bool qsplit = false;           // the sparse list holds the SMALL groups (query-lane rule): only the
                                   // device single pass uses it (k_qlanes); other paths ignore the split
    uint64_t tests_total = 0;      // sum over groups of queries x candidates (0: not computed); >= P
    cudaStream_t stream = nullptr; // stream the buffers were allocated on
    float ms_build = 0;
};

// ---------------------------------------------------------------- kernels
// grid build (kernels_grid.cu)
// bbox sentinels bb[0..3], zeroes bb[4..nz); with hkey: the occupancy hash table (tsize entries)
void launch_bbox_init(unsigned long long* bb, uint32_t nz, unsigned long long* hkey, unsigned int* hcnt,
                      uint32_t tsize, cudaStream_t s);
// the grid build's readbacks in one place: out[0..5] = *ng, *mw, *dn, *sn, sp[0], sp[1] (null -> 0)
void launch_readback(unsigned long long* out, const uint32_t* ng, const uint64_t* mw, const uint32_t* dn,
                     const uint32_t* sn, const unsigned long long* sp, cudaStream_t s);
void launch_bbox(const void* xy, uint64_t n, hdb_dtype dt, unsigned long long* bb, unsigned int* bad,
                 cudaStream_t s);
double bbox_decode(unsigned long long v, bool is_max);
size_t radix_sort_temp_bytes(uint64_t n);
// Stable LSD radix sort of (keys, vals) on the low `bits` bits.  Ping-pongs
// between (k0,v0) and (k1,v1); returns 0 if the result is in (k0,v0), 1 else.
int radix_sort_pairs(void* k0, uint32_t* v0, void* k1, uint32_t* v1, int key_bytes, uint64_t n, int bits,
                     void* temp, cudaStream_t s);
// a2 + a3 + gather: the points sorted by cell key (stable LSD radix sort of (key, id, xy)
// records, keys computed by the first pass from the input points): keys_out[n] sorted keys,
// ids_out[n + 2] A (padded), xy_s[n + 2] sorted points (padded), xp the f32 filter copy
// (padded), counters zeroed.  temp: point_sort_temp_bytes(n, dt, key_bytes, bits)
// process-shard bands: one pass over the input -> every point's cell row
// (rowid[n]), exact row counts row_cnt[ny] (zeroed by the caller) and, with cell_cnt (a
// zeroed nx*ny histogram of a 1/16 sample), row_load[ny] = the estimated sum of squared cell
// counts x 256; the band's points (rowid in [ylo, yhi)) with their input rows; the band's
// query groups (cells with keys in [key_lo, key_hi)) -> out[0..1]
void band_rows_hist(const void* xy, uint64_t n, hdb_dtype dt, double xmin, double ymin, double inv_w, uint32_t nx,
                    uint32_t ny, uint32_t* rowid, uint32_t* cell_cnt, unsigned long long* row_cnt,
                    unsigned long long* row_load, cudaStream_t s);
void band_select(const void* xy, const uint32_t* rowid, uint64_t n, hdb_dtype dt, uint64_t ylo, uint64_t yhi, void* out,
                 uint32_t* gid, uint32_t* n_out, void* temp, cudaStream_t s);
void launch_band_groups(const uint64_t* ckey, uint64_t nne, const uint32_t* gofs, uint64_t key_lo, uint64_t key_hi,
                        unsigned long long* out, cudaStream_t s);
size_t point_sort_temp_bytes(uint64_t n, hdb_dtype dt, int key_bytes, int bits);
// gid (optional): the points' ids (a process shard's band of the input); else the input row
void sort_points(const void* xy_in, uint64_t n, hdb_dtype dt, double xmin, double ymin, double inv_w, uint32_t nx,
                 uint32_t ny, int key_bytes, int bits, void* keys_out, uint32_t* ids_out, void* xy_s, float4* xp,
                 double ox, double oy, unsigned int* counters, uint32_t n_counters, void* temp, cudaStream_t s,
                 const uint32_t* gid = nullptr);
// cnext: optional dense lookup (first non-empty cell with key >= h, h in [0, nx*ny]); null = binary search
void launch_cell_spans(const uint64_t* ckey, const uint32_t* cstart, uint64_t nne, uint32_t nx, uint32_t ny,
                       uint32_t k, uint2* cspan, uint32_t* gcount, const uint32_t* cnext, cudaStream_t s);
// mark[ckey[c]] = 1 for every non-empty cell (mark zeroed by the caller)
void launch_cell_mark(const uint64_t* ckey, uint64_t nne, uint32_t* mark, cudaStream_t s);
// auto cell split: sample-based point-weighted occupancy at cell width 1/inv_w;
// out[0] = sum s_c (s_c - 1), out[1] = sum s_c over the sampled cells
void launch_occ_estimate(const void* xy, uint64_t n, hdb_dtype dt, uint64_t stride, uint64_t m, double inv_w,
                         unsigned long long* hkey, unsigned int* hcnt, uint32_t tsize, unsigned long long* out,
                         cudaStream_t s);
void launch_group_build(const uint32_t* cstart, const uint32_t* gofs, uint64_t nne, uint64_t n, uint32_t* gstart,
                        uint32_t* gcell, cudaStream_t s);
// dense/sparse classification of the groups g < *ng_dev (entries up to n): dflag[g] = 1 for a
// dense group, sqn[g] = its query count for a sparse one (sparse <=> queries x candidates <=
// max_tests), n_sparse[0] += the sparse queries, n_sparse[1] += every group's candidate tests; then the lists dl[dpre[g]] = g (dense) and
// sql[spre[g] + i] = {gstart[g] + i, gcell[g]}
void launch_group_class(const uint32_t* cstart, const uint2* cspan, uint32_t nspan, const uint32_t* gstart,
                        const uint32_t* gcell, const uint32_t* ng_dev, uint64_t n, uint32_t max_tests,
                        bool qlanes, uint32_t* dflag, uint32_t* sqn, unsigned long long* n_sparse, uint8_t* gbin,
                        uint32_t* ohist, uint32_t* words, uint32_t win, cudaStream_t s);
// cost order: ord = the groups by gbin (dense groups first, heaviest first); ohist holds
// 2 * kOrderBins words (bin sizes from launch_group_class, then cursors; zeroed by the caller);
// launch_group_class also writes the hit-mask words per group (windows of win chunks)
constexpr int kOrderBins = 64;
#ifndef HDB_KWIN
#define HDB_KWIN 8
#endif
constexpr int kMaskWin = HDB_KWIN;   // chunks per window of the hit-mask layout (kernels_search.cu kWin)
void launch_order_scatter(const uint8_t* gbin, const uint32_t* ng_dev, uint64_t n, uint32_t* ohist, uint32_t* ord,
                          cudaStream_t s);
void launch_group_lists(const uint32_t* gstart, const uint32_t* gcell, const uint32_t* ng_dev, uint64_t n,
                        const uint32_t* dpre, const uint32_t* spre, uint32_t* dl, uint2* sql, bool qlanes,
                        cudaStream_t s);

// scans (kernels_scan.cu): exclusive scan of in[0..n) into out[0..n], out[n] = total
size_t scan_temp_bytes(uint64_t n);
// Per-device tile-status buffer for memset-free scans (zeroed once, one epoch per scan).
// Scans issued by a thread while a ScanEpochScope is alive use it (all on one stream: the
// scans of one scope must not run concurrently); others zero their status tiles in temp.
struct ScanEpochs {
    unsigned long long* tiles = nullptr;   // cap tile words + the tile-id counter (tiles[cap])
    uint64_t cap = 0;      // tiles
    uint32_t epoch = 0;    // last epoch used
    uint64_t ctr_base = 0; // tile ids handed out so far by tiles[cap] (scans in stream order)
};
extern thread_local ScanEpochs* t_scan_epochs;
struct ScanEpochScope {
    ScanEpochs* prev;
    explicit ScanEpochScope(ScanEpochs* e) : prev(t_scan_epochs) { t_scan_epochs = e; }
    ~ScanEpochScope() { t_scan_epochs = prev; }
};
void scan_u32_to_u32(const uint32_t* in, uint32_t* out, uint64_t n, void* temp, cudaStream_t s);
void scan_u32_to_u64(const uint32_t* in, uint64_t* out, uint64_t n, void* temp, cudaStream_t s);
// a4: run-length encoding of n sorted cell keys (one look-back scan of the run-start flags):
// ckey[c], cstart[c] for every non-empty cell c, cstart[nne] = n, *nne_out = nne.
// ckey / cstart must hold n / n + 1 entries (nne <= n is known only after the call)
void cell_rle(const void* keys_sorted, int key_bytes, uint64_t n, uint64_t* ckey, uint32_t* cstart, uint32_t* nne_out,
              void* temp, cudaStream_t s);

// search (kernels_search.cu)
// Sampled count (a5): |N_eps| of sorted positions j*stride, j < n_sample -> samp_cnt, sum.
void launch_sample_count(const DevGrid& g, uint64_t stride, uint64_t n_sample, uint32_t* samp_cnt,
                         unsigned long long* sum, cudaStream_t s);
// Exact count (a6) over query groups [g0, g1): cnt[sorted pos].
// masks (optional): the hit-mask table (see k_emit), laid out by g.moff.
void launch_count(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests,
                  int variant, int slot, uint2* masks, cudaStream_t s);
// Write (a8) over groups [g0, g1): out[off[q] - out_base + k] = k-th neighbour id of q.
// masks != null: emit from the stored hit masks; null: recompute the tests.
// single-pass device table (k_fused): count + reserve + emit per group; mask
// table `masks` laid out by g.moff; rows reserved on *pair_ctr (zeroed by the
// caller); *overflow set if a reservation passed cap
// over the query groups [g0, g1) (a process shard's band: its range); cnt may be null
void launch_fused(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests, uint2* masks,
                  unsigned long long* pair_ctr, uint64_t cap, uint32_t* out, uint64_t* begin, uint32_t* count,
                  unsigned int* overflow, cudaStream_t s, bool pos_out = false);
// single pass for the sparse queries (dense/sparse split): thread per query, rows reserved
// on the same pair counter as launch_fused (run both on one stream)
void launch_sparse_fused(const DevGrid& g, uint64_t g0, uint64_t g1, unsigned long long* tests,
                         unsigned long long* pair_ctr, uint64_t cap, uint32_t* out, uint64_t* begin, uint32_t* count,
                         unsigned int* overflow, cudaStream_t s, bool pos_out = false);
void launch_write(const DevGrid& g, uint64_t g0, uint64_t g1, const uint64_t* off, uint64_t out_base,
                  uint32_t* out, int variant, int slot, const uint2* masks, cudaStream_t s,
                  uint64_t* begin = nullptr, uint32_t* count = nullptr);
// words[g] = 32-bit words of group g's hit masks for g < *ng_dev, 0 for g in [*ng_dev, n) (scan -> g.moff)
void launch_mask_words(const DevGrid& g, const uint32_t* ng_dev, uint64_t n, uint32_t* words, cudaStream_t s);
// cuts: for b in 0..nb, gcut[b] = first group g in [g0,g1] with off[gstart[g]] >= target_b,
// target_b = off[gstart[g0]] + b * span / nb (gcut[0] = g0, gcut[nb] = g1); pcut[b] = off[gstart[gcut[b]]]
void launch_batch_cuts(const uint32_t* gstart, const uint64_t* off, uint64_t g0, uint64_t g1, uint32_t nb,
                       uint64_t* gcut, uint64_t* pcut, cudaStream_t s);
// map sorted positions -> the first group starting at or after them (binary search in gstart)
void launch_pos_to_group(const uint32_t* gstart, uint64_t n_groups, const uint64_t* pos, uint32_t m,
                         uint64_t* grp, cudaStream_t s);
// DBSCAN on a device-resident table (kernels_dbscan.cu); rank[n] = number of clusters
// rows: the table's production order (cell-sorted queries), or null
void launch_dbscan_device(const uint64_t* begin, const uint32_t* count, const uint32_t* nbrs, const uint32_t* rows,
                          uint64_t n, uint64_t npairs, uint32_t minpts, uint8_t* core, uint32_t* parent,
                          uint32_t* root, uint32_t* is_root, uint32_t* rank, uint32_t* giant, uint32_t* bits,
                          uint32_t* sched /* 2 x SM count */, uint64_t* pre /* n + 1 */, void* scan_temp,
                          int32_t* labels, cudaStream_t s, bool pos_space = false,
                          uint8_t* core_out = nullptr);

// the paper's kernels (kernels_paper.cu; search_kernel 7 / 8):
// the key/value result set R of GPUCalcGlobal (Alg. 2) or GPUCalcShared (Alg. 3),
// appended at *ctr (zeroed by the caller; counts past cap, writes only below it)
constexpr int kPaperGlobal = 7, kPaperShared = 8;
void launch_paper_search(const DevGrid& g, int which, unsigned long long* ctr, uint64_t cap, uint32_t* rkey,
                         uint32_t* rval, cudaStream_t s);
// T ranges from R sorted by key: begin[k] = first position of key k, count[k] = its run length
void launch_rows_from_keys(const uint32_t* key_sorted, uint64_t m, uint64_t n, uint64_t* begin, uint32_t* count,
                           cudaStream_t s);

// ---------------------------------------------------------------- pools
struct PinnedPool {
    std::mutex m;
    std::multimap<size_t, void*> free_blocks;
    size_t bytes_total = 0;
    uint64_t grows = 0;
    void* acquire(size_t bytes, size_t* got);
    void release(void* p, size_t bytes);
    ~PinnedPool();
};

struct DevCtx {
    int device = 0;
    cudaStream_t main = nullptr;
    bool own_main = true;
    std::vector<cudaStream_t> streams;     // write + D2H streams
    std::vector<cudaEvent_t> ev_pool;
    uint64_t* pin = nullptr;                // small pinned scratch for async readbacks
    // Stream-ordered pool of its own for the table-sized buffers (neighbour lists,
    // hit masks, T by id): step-sized blocks then reuse each other instead of
    // being carved up by the grid's smaller buffers in the default pool (which
    // made C5 steps map fresh memory: 27 -> 60..120 ms outliers)
    cudaMemPool_t big_pool = nullptr;
    size_t total_mem = 0;                   // device memory (bytes), for sizing decisions
    ScanEpochs scan_ep;                     // memset-free scans of the grid build / count phase
    // cached per-stream device batch buffers (reused across calls)
    std::vector<uint32_t*> batch_buf;
    std::vector<size_t> batch_cap;
};

}  // namespace hdb

struct hdb_ctx {
    hdb_opts opts{};
    std::vector<int> device_list;
    std::vector<hdb::DevCtx> dev;
    std::shared_ptr<hdb::PinnedPool> pinned;
    std::recursive_mutex mu;
    hdb_stats stats{};
    std::atomic<int> live_objects{0};
};

struct hdb_grid {
    hdb_ctx* ctx = nullptr;
    std::vector<hdb::DevGrid> dev;   // one per ctx device (same content)
};

struct hdb_table {
    uint64_t n = 0, npairs = 0;
    double eps = 0;
    hdb_dtype dtype = HDB_F64;
    bool on_device = false;
    int device = 0;
    uint64_t first_query = 0, end_query = 0;
    uint64_t* begin = nullptr;
    uint32_t* count = nullptr;
    uint32_t* nbrs = nullptr;
    uint32_t* rows = nullptr;   // device tables only: query ids in production (cell-sorted) order
    // position space (internal tables of the device sweep only, never handed to the caller):
    // nbrs hold sorted POSITIONS and begin / count are indexed by position; rows[pos] = id
    bool pos_space = false;
    // ownership
    std::shared_ptr<hdb::PinnedPool> pool;   // non-null: begin/count/nbrs are pinned pool blocks
    size_t cap_begin = 0, cap_count = 0, cap_nbrs = 0;
    bool malloced = false;                   // begin/count/nbrs from malloc
    cudaStream_t dstream = nullptr;          // device-resident: stream for cudaFreeAsync
    int host_threads = 0;
    hdb_ctx* ctx = nullptr;
};

namespace hdb {
int resolve_threads(int requested);
// engine.cpp
void grid_build(hdb_ctx* ctx, const void* xy, uint64_t n, hdb_dtype dt, double eps, hdb_grid** out);
void grid_free(hdb_grid* g);
// pos_space: a device-resident table in position space if the single pass builds it (DESIGN.md
// "position space"); otherwise (two-pass fallback) an ordinary id-space table
void neighbor_table(hdb_ctx* ctx, const hdb_grid* grid, bool device_resident, hdb_table** out,
                    bool pos_space = false);
void table_free(hdb_table* t);
// dbscan.cpp
uint32_t dbscan_host(const hdb_table* t, uint32_t minpts, int n_threads, int32_t* labels, uint8_t* core);
uint32_t dbscan_device(const hdb_table* t, uint32_t minpts, int32_t* labels, uint8_t* core);
bool is_device_ptr(const void* p);   // CUDA device / managed memory
void canonicalize(hdb_table* t);
}  // namespace hdb
