// kernels_scan.cu -- device exclusive scans (SURVEY 8(a) a4 cell offsets, a7
// neighbour-list offsets).  One pass over 4096-element tiles; inside a tile
// every thread scans 16 consecutive items serially, the warp combines its lanes
// with __shfl_up_sync and the CTA combines its 8 warp totals; tiles chain their
// prefixes by decoupled look-back.  out[n] receives the total.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace hdb {

std::atomic<uint64_t> g_kernel_launches{0};

namespace {

constexpr unsigned FULL = 0xffffffffu;
#ifndef HDB_SC_ITEMS
#define HDB_SC_ITEMS 16   // tiles of 4,096: C5 run-length encoding 354 -> 258 us, 7 plain scans 273 -> 198 us
#endif
#ifndef HDB_SC_ITEMS32
#define HDB_SC_ITEMS32 16  // 32 (tiles of 8,192): C5 / C2 unchanged, C3 -2% (A/B profiles/r2q) -- kept at 16
#endif
constexpr int SC_THREADS = 256;
// items per thread: fewer, longer tiles shorten the look-back chains (latency-bound)
template <typename Tout>
struct Sc {
    static constexpr int ITEMS = sizeof(Tout) == 4 ? HDB_SC_ITEMS32 : HDB_SC_ITEMS;
    static constexpr int TILE = SC_THREADS * ITEMS;
};
constexpr int SC_TILE_MIN = SC_THREADS * (HDB_SC_ITEMS < HDB_SC_ITEMS32 ? HDB_SC_ITEMS : HDB_SC_ITEMS32);

// Single-pass scan with decoupled look-back (Merrill & Garland 2016): tile t
// publishes its aggregate, then its inclusive prefix once known, as one packed
// 64-bit word {status:2, value:62}; a tile finds its exclusive prefix by walking
// back over its predecessors' words, 32 at a time (one per lane of warp 0),
// summing aggregates until it meets an inclusive prefix.  A CTA takes its tile
// index from an atomic counter when it starts (not blockIdx.x: the CUDA model
// does not promise dispatch in blockIdx order), so a tile only ever waits on
// tiles whose CTAs are already running -- no deadlock under concurrent kernels
// or MPS.  The counter is never reset: a scan's tiles are the counter values
// [ctr_base, ctr_base + nb), ctr_base tracked on the host (stream order).
// One kernel per scan (plus a memset of the tile words on the memset path).
// Tile status word: flag (2 bits: aggregate / inclusive prefix) | epoch (20 bits) | value (42 bits).
// A word is ready only with a flag and the scan's own epoch: memset-path scans use epoch 0 on a
// zeroed buffer; epoch scans (ScanEpochScope) reuse one zeroed per-device buffer with a new
// epoch per call and need no memset.  Values stay < 2^42 (counts of points / pairs / mask words
// bounded by device memory).
constexpr uint64_t kStAgg = 1ull << 62, kStPre = 2ull << 62, kValMask = (1ull << 42) - 1;
constexpr int kEpShift = 42;
constexpr uint64_t kEpMask = (1ull << 20) - 1;

__device__ __forceinline__ void publish(unsigned long long* w, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(w), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t peek(const unsigned long long* w) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(w) : "memory");
    return v;
}

// Op: Tout load(idx) (idx < n) -- the item; void store(idx, excl, item) -- its exclusive prefix
// (and the item again, recovered from the prefixes -- the load is not repeated);
// void total(t) -- the sum of all items (written by the last tile)
template <typename Tin, typename Tout>
struct PlainScan {
    const Tin* __restrict__ in;
    Tout* __restrict__ out;
    __device__ __forceinline__ Tout load(uint64_t i) const { return (Tout)in[i]; }
    __device__ __forceinline__ void store(uint64_t i, Tout e, Tout) const { out[i] = e; }
    __device__ __forceinline__ void total(uint64_t n, Tout t) const { out[n] = t; }
};

template <typename Tout, typename Op>
__global__ void __launch_bounds__(SC_THREADS) k_scan_lookback(Op op, uint64_t n, unsigned long long* __restrict__ tiles,
                                                              uint64_t ep, unsigned long long* __restrict__ ctr,
                                                              uint64_t ctr_base) {
    constexpr int SC_ITEMS = Sc<Tout>::ITEMS, SC_TILE = Sc<Tout>::TILE;
    // one pad word per 32: the per-thread runs (stride SC_ITEMS) are bank-conflict free
    __shared__ Tout buf[SC_TILE + SC_TILE / 32];
    auto bi = [](int j) { return j + (j >> 5); };
    __shared__ Tout wsum[SC_THREADS / 32];
    __shared__ Tout s_excl;
    __shared__ uint64_t s_tile;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    if (tid == 0) s_tile = ctr ? atomicAdd(ctr, 1ull) - ctr_base : 0;
    __syncthreads();
    const uint64_t t = s_tile;
    const uint64_t base = t * SC_TILE;
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        uint64_t idx = base + (uint64_t)i * SC_THREADS + tid;
        buf[bi(i * SC_THREADS + tid)] = idx < n ? op.load(idx) : (Tout)0;
    }
    __syncthreads();
    Tout v[SC_ITEMS];
    Tout run = 0;
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        v[i] = run;
        run += buf[bi(tid * SC_ITEMS + i)];
    }
    Tout incl = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        Tout y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) wsum[w] = incl;
    __syncthreads();
    Tout wpre = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < SC_THREADS / 32; ++i) {
        Tout x = wsum[i];
        wpre += (i < w) ? x : (Tout)0;
        tot += x;
    }
    // Look-back by the whole CTA: 256 predecessors per step (a warp looking at 32 per step
    // walked back through a whole wave of concurrently started tiles -- ~900 aggregates,
    // ~28 dependent L2 round trips -- while the other warps waited at the barrier)
    __shared__ int s_first;
    __shared__ Tout s_lb[SC_THREADS / 32];
    Tout excl = 0;
    if (t == 0) {
        if (tid == 0 && tiles) publish(&tiles[0], kStPre | ep | (uint64_t)tot);
    } else {
        if (tid == 0) publish(&tiles[t], kStAgg | ep | (uint64_t)tot);
        // before tile 0: prefix 0; a word of another epoch counts as not yet published
        auto ready = [&](uint64_t wd) { return (wd >> 62) != 0 && (wd & (kEpMask << kEpShift)) == ep; };
        int64_t pred = (int64_t)t - 1;
        while (true) {
            const int64_t j = pred - tid;
            uint64_t word = j >= 0 ? peek(&tiles[j]) : (kStPre | ep);
            while (__syncthreads_or(!ready(word))) {   // wait for every predecessor in view
                if (!ready(word)) word = peek(&tiles[j]);
            }
            if (tid == 0) s_first = SC_THREADS;
            __syncthreads();
            if ((word >> 62) == 2) atomicMin(&s_first, tid);   // nearest inclusive prefix
            __syncthreads();
            const int first = s_first;
            Tout val = tid <= first ? (Tout)(word & kValMask) : (Tout)0;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) val += __shfl_xor_sync(FULL, val, o);
            if (lane == 0) s_lb[w] = val;
            __syncthreads();
#pragma unroll
            for (int i = 0; i < SC_THREADS / 32; ++i) excl += s_lb[i];
            if (first < SC_THREADS) break;
            pred -= SC_THREADS;
            __syncthreads();   // s_first / s_lb are rewritten by the next step
        }
        if (tid == 0) publish(&tiles[t], kStPre | ep | (uint64_t)(excl + tot));
    }
    if (tid == 0) s_excl = excl;
    __syncthreads();
    const Tout pre = s_excl + wpre + (incl - run);
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) buf[bi(tid * SC_ITEMS + i)] = pre + v[i];
    __syncthreads();
    const Tout tile_end = s_excl + tot;   // inclusive prefix of the tile's last item
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        const int j = i * SC_THREADS + tid;
        uint64_t idx = base + (uint64_t)j;
        if (idx < n) {
            // the item itself = the next position's exclusive prefix - this one's
            const Tout e = buf[bi(j)];
            op.store(idx, e, (j + 1 < SC_TILE ? buf[bi(j + 1)] : tile_end) - e);
        }
    }
    if (tid == 0 && base + SC_TILE >= n) op.total(n, s_excl + tot);   // last tile writes the total
}

template <typename Tout, typename Op>
void scan_impl(const Op& op, uint64_t n, void* temp, cudaStream_t s) {
    constexpr int SC_TILE = Sc<Tout>::TILE;
    const uint64_t nb = (n + SC_TILE - 1) / SC_TILE;
    unsigned long long* tiles = nullptr;
    unsigned long long* ctr = nullptr;   // tile-id counter (null: one tile, id 0)
    uint64_t ep = 0, ctr_base = 0;
    if (nb > 1) {
        ScanEpochs* se = t_scan_epochs;
        if (se && nb <= se->cap) {
            if (++se->epoch > kEpMask) {   // epochs wrap: start again on a zeroed buffer (+ counter)
                cudaMemsetAsync(se->tiles, 0, (se->cap + 1) * sizeof(unsigned long long), s);
                se->epoch = 1;
                se->ctr_base = 0;
            }
            tiles = se->tiles;
            ctr = se->tiles + se->cap;
            ctr_base = se->ctr_base;
            se->ctr_base += nb;
            ep = (uint64_t)se->epoch << kEpShift;
        } else {
            tiles = (unsigned long long*)temp;
            ctr = tiles + nb;
            cudaMemsetAsync(tiles, 0, (nb + 1) * sizeof(unsigned long long), s);
        }
    }
    k_scan_lookback<Tout, Op><<<(unsigned)nb, SC_THREADS, 0, s>>>(op, n, tiles, ep, ctr, ctr_base);
    ++g_kernel_launches;
}

}  // namespace

thread_local ScanEpochs* t_scan_epochs = nullptr;

size_t scan_temp_bytes(uint64_t n) {
    return ((n + SC_TILE_MIN - 1) / SC_TILE_MIN + 2) * sizeof(unsigned long long) + 64;   // tile words + counter
}

void scan_u32_to_u32(const uint32_t* in, uint32_t* out, uint64_t n, void* temp, cudaStream_t s) {
    if (n == 0) {
        cudaMemsetAsync(out, 0, sizeof(uint32_t), s);
        return;
    }
    scan_impl<uint32_t>(PlainScan<uint32_t, uint32_t>{in, out}, n, temp, s);
}

void scan_u32_to_u64(const uint32_t* in, uint64_t* out, uint64_t n, void* temp, cudaStream_t s) {
    if (n == 0) {
        cudaMemsetAsync(out, 0, sizeof(uint64_t), s);
        return;
    }
    scan_impl<uint64_t>(PlainScan<uint32_t, uint64_t>{in, out}, n, temp, s);
}

// a4 in one pass: run-length encoding of the sorted keys -- the scan of the run-start
// flags (key[s] != key[s-1]) gives each run its index c; run starts write ckey[c] = key,
// cstart[c] = s; the total (the non-empty cell count) goes to cstart's terminator slot
// *nne_out and cstart[nne] = n is written by the last tile.  Replaces flags -> scan ->
// scatter (three passes over n-sized arrays).
template <typename K>
struct RleScan {
    const K* __restrict__ keys;
    uint64_t* __restrict__ ckey;
    uint32_t* __restrict__ cstart;
    uint32_t* __restrict__ nne_out;
    __device__ __forceinline__ uint32_t load(uint64_t i) const {
        return (i == 0 || keys[i] != keys[i - 1]) ? 1u : 0u;
    }
    __device__ __forceinline__ void store(uint64_t i, uint32_t e, uint32_t run_start) const {
        if (run_start) {
            ckey[e] = (uint64_t)keys[i];
            cstart[e] = (uint32_t)i;
        }
    }
    __device__ __forceinline__ void total(uint64_t n, uint32_t t) const {
        cstart[t] = (uint32_t)n;
        *nne_out = t;
    }
};

// process-shard band: the points whose cell row (rowid, from the band
// histogram pass) is in [ylo, yhi), in input order, with their input rows (stream
// compaction as a scan of the membership flags; only members' coordinates are read)
template <typename P2>
struct BandSelect {
    const P2* __restrict__ xy;
    const uint32_t* __restrict__ rowid;
    uint64_t ylo, yhi;
    P2* __restrict__ out;
    uint32_t* __restrict__ gid;
    uint32_t* __restrict__ n_out;
    __device__ __forceinline__ uint32_t load(uint64_t i) const {
        const uint32_t y = rowid[i];
        return y >= ylo && y < yhi ? 1u : 0u;
    }
    __device__ __forceinline__ void store(uint64_t i, uint32_t e, uint32_t member) const {
        if (member) {
            out[e] = xy[i];
            gid[e] = (uint32_t)i;
        }
    }
    __device__ __forceinline__ void total(uint64_t, uint32_t t) const { *n_out = t; }
};

void band_select(const void* xy, const uint32_t* rowid, uint64_t n, hdb_dtype dt, uint64_t ylo, uint64_t yhi, void* out,
                 uint32_t* gid, uint32_t* n_out, void* temp, cudaStream_t s) {
    if (n == 0) {
        cudaMemsetAsync(n_out, 0, sizeof(uint32_t), s);
        return;
    }
    if (dt == HDB_F64)
        scan_impl<uint32_t>(BandSelect<double2>{(const double2*)xy, rowid, ylo, yhi, (double2*)out, gid, n_out}, n,
                            temp, s);
    else
        scan_impl<uint32_t>(BandSelect<float2>{(const float2*)xy, rowid, ylo, yhi, (float2*)out, gid, n_out}, n, temp,
                            s);
}

void cell_rle(const void* keys_sorted, int key_bytes, uint64_t n, uint64_t* ckey, uint32_t* cstart, uint32_t* nne_out,
              void* temp, cudaStream_t s) {
    if (n == 0) {
        cudaMemsetAsync(cstart, 0, sizeof(uint32_t), s);
        cudaMemsetAsync(nne_out, 0, sizeof(uint32_t), s);
        return;
    }
    if (key_bytes == 4)
        scan_impl<uint32_t>(RleScan<uint32_t>{(const uint32_t*)keys_sorted, ckey, cstart, nne_out}, n, temp, s);
    else
        scan_impl<uint32_t>(RleScan<uint64_t>{(const uint64_t*)keys_sorted, ckey, cstart, nne_out}, n, temp, s);
}

}  // namespace hdb
