// dbscan.cpp -- host DBSCAN on the neighbour table T.
//
// The paper's "modified DBSCAN": Alg. 1 with the index
// searches of lines 9 and 18 replaced by lookups in T, so only minpts remains
// a parameter and one T serves every minpts.  Output follows the
// canonical rule (R7), which is exactly what Alg. 1 produces when run
// over p = 0..n-1:
//   core(p)  <=> |N_eps(p)| >= minpts (count includes p)
//   clusters  = components of the core-core graph, numbered by increasing
//               minimum core id (the order Alg. 1 line 24 appends them)
//   border p -> the lowest-numbered cluster among its core neighbours (the first
//               cluster whose expansion reaches p)
//   noise     = everything else, label -1.
// Two implementations with identical output:
//   * sequential: cluster-at-a-time BFS over cores in id order (n_threads == 1);
//   * parallel:   lock-free union-find over core-core edges with min-id roots
//                 (Afforest-style sampled links, then the lists of the two
//                 giant components skipped by the rule in dbscan_par, as the
//                 device code), root ranks by a prefix count, borders by a min
//                 over core neighbours (NEXT-2; the paper runs variants, not one
//                 variant, in parallel).
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <atomic>
#include <cstring>
#include <memory>
#include <thread>
#include <vector>

#include "internal.h"

namespace hdb {

namespace {

uint32_t dbscan_seq(const hdb_table* t, uint32_t minpts, int32_t* labels, uint8_t* core) {
    const uint64_t n = t->n;
    const uint64_t* B = t->begin;
    const uint32_t* C = t->count;
    const uint32_t* V = t->nbrs;
    for (uint64_t p = 0; p < n; ++p) {
        labels[p] = -1;
        core[p] = C[p] >= minpts ? 1 : 0;
    }
    std::vector<uint32_t> stack;
    int32_t k = 0;
    for (uint64_t p = 0; p < n; ++p) {
        if (!core[p] || labels[p] != -1) continue;
        labels[p] = k;
        stack.clear();
        stack.push_back((uint32_t)p);
        while (!stack.empty()) {
            uint32_t u = stack.back();
            stack.pop_back();
            const uint32_t* L = V + B[u];
            for (uint32_t i = 0, m = C[u]; i < m; ++i) {
                uint32_t v = L[i];
                if (labels[v] == -1) {
                    labels[v] = k;
                    if (core[v]) stack.push_back(v);
                }
            }
        }
        ++k;
    }
    return (uint32_t)k;
}

inline uint32_t uf_find(std::atomic<uint32_t>* parent, uint32_t x) {
    uint32_t p = parent[x].load(std::memory_order_relaxed);
    while (p != x) {
        uint32_t gp = parent[p].load(std::memory_order_relaxed);
        if (gp != p) parent[x].compare_exchange_weak(p, gp, std::memory_order_relaxed);  // path halving
        x = p;
        p = parent[x].load(std::memory_order_relaxed);
    }
    return x;
}

// link the larger root under the smaller: every root stays its tree's minimum id
inline void uf_union(std::atomic<uint32_t>* parent, uint32_t a, uint32_t b) {
    while (true) {
        a = uf_find(parent, a);
        b = uf_find(parent, b);
        if (a == b) return;
        if (a < b) std::swap(a, b);   // a > b: hang a under b
        uint32_t expect = a;
        if (parent[a].compare_exchange_strong(expect, b, std::memory_order_relaxed)) return;
    }
}

template <typename F>
void parallel_for(int T, uint64_t n, F&& f) {
    if (T <= 1 || n < 4096) {
        f(0, n, 0);
        return;
    }
    std::vector<std::thread> th;
    uint64_t chunk = (n + T - 1) / T;
    for (int k = 0; k < T; ++k) {
        uint64_t a = k * chunk, b = std::min<uint64_t>(n, a + chunk);
        if (a >= b) break;
        th.emplace_back([&, a, b, k] { f(a, b, k); });
    }
    for (auto& x : th) x.join();
}

uint32_t dbscan_par(const hdb_table* t, uint32_t minpts, int T, int32_t* labels, uint8_t* core) {
    // HDB_TRACE=1: wall time of each phase, to stderr
    const char* tre = std::getenv("HDB_TRACE");
    const bool trace = tre && *tre == '1';
    auto tlast = std::chrono::steady_clock::now();
    std::string tlog;
    auto mark = [&](const char* what) {
        if (!trace) return;
        const auto now = std::chrono::steady_clock::now();
        char buf[96];
        snprintf(buf, sizeof buf, " %s=%.2f", what, std::chrono::duration<double, std::milli>(now - tlast).count());
        tlog += buf;
        tlast = now;
    };
    const uint64_t n = t->n;
    const uint64_t* B = t->begin;
    const uint32_t* C = t->count;
    const uint32_t* V = t->nbrs;
    std::unique_ptr<std::atomic<uint32_t>[]> parent(new std::atomic<uint32_t>[n ? n : 1]);
    parallel_for(T, n, [&](uint64_t a, uint64_t b, int) {
        for (uint64_t p = a; p < b; ++p) {
            core[p] = C[p] >= minpts ? 1 : 0;
            parent[p].store((uint32_t)p, std::memory_order_relaxed);
        }
    });
    mark("init");
    // Afforest-style pre-pass (as the device code): two rounds of one sampled
    // link per core, each followed by a compression of every core to its root.
    // The sampled list entry and then its parent / core flag are two dependent random reads
    // per core (ids are a random permutation of space): software prefetch, the list entry
    // 2 D iterations ahead and its parent / core flag D ahead, keeps ~2 D misses in flight
    // per thread instead of one.
    constexpr uint64_t D = 16;
    for (uint32_t k = 1; k <= 2; ++k) {
        parallel_for(T, n, [&](uint64_t a, uint64_t b, int) {
            for (uint64_t u = a; u < b; ++u) {
                if (u + 2 * D < b) {
                    const uint64_t w = u + 2 * D;
                    __builtin_prefetch(&V[B[w] + (uint64_t)C[w] * k / 3]);
                }
                if (u + D < b) {
                    const uint64_t w = u + D;
                    if (core[w] && C[w]) {
                        const uint32_t vw = V[B[w] + (uint64_t)C[w] * k / 3];
                        __builtin_prefetch(&parent[vw]);
                        __builtin_prefetch(&core[vw]);
                    }
                }
                if (!core[u] || C[u] == 0) continue;
                const uint32_t v = V[B[u] + (uint64_t)C[u] * k / 3];
                if (v != u && core[v]) uf_union(parent.get(), (uint32_t)u, v);
            }
        });
        parallel_for(T, n, [&](uint64_t a, uint64_t b, int) {
            for (uint64_t p = a; p < b; ++p)
                if (core[p]) parent[p].store(uf_find(parent.get(), (uint32_t)p), std::memory_order_relaxed);
        });
    }
    mark("sample_links");
    // the two most frequent roots among 1024 sampled points (>= 1/8 of them):
    // giant components A and B, with membership bitmaps
    const uint32_t kNone = 0xffffffffu;
    uint32_t gA = kNone, gB = kNone;
    if (n >= 4096) {
        std::vector<uint32_t> smp;
        for (uint64_t i = 0; i < 1024; ++i) {
            const uint64_t p = i * n / 1024;
            if (core[p]) smp.push_back(uf_find(parent.get(), (uint32_t)p));
        }
        std::sort(smp.begin(), smp.end());
        std::vector<std::pair<uint32_t, uint32_t>> runs;   // (count, root)
        for (size_t i = 0; i < smp.size();) {
            size_t j = i;
            while (j < smp.size() && smp[j] == smp[i]) ++j;
            runs.emplace_back((uint32_t)(j - i), smp[i]);
            i = j;
        }
        std::sort(runs.begin(), runs.end(), std::greater<>());
        if (runs.size() > 0 && runs[0].first >= 128) gA = runs[0].second;
        if (runs.size() > 1 && runs[1].first >= 128) gB = runs[1].second;
    }
    const uint64_t nw = (n + 63) / 64;
    std::vector<uint64_t> bitA(gA != kNone ? nw : 0), bitB(gB != kNone ? nw : 0);
    if (gA != kNone) {
        parallel_for(T, nw, [&](uint64_t a, uint64_t b, int) {
            for (uint64_t w = a; w < b; ++w) {
                uint64_t ma = 0, mb = 0;
                for (uint64_t p = 64 * w; p < std::min(n, 64 * w + 64); ++p) {
                    if (!core[p]) continue;
                    const uint32_t r = uf_find(parent.get(), (uint32_t)p);
                    if (r == gA) ma |= 1ull << (p & 63);
                    if (r == gB) mb |= 1ull << (p & 63);
                }
                bitA[w] = ma;
                if (gB != kNone) bitB[w] = mb;
            }
        });
    }
    auto inA = [&](uint32_t v) { return gA != kNone && ((bitA[v >> 6] >> (v & 63)) & 1); };
    auto inB = [&](uint32_t v) { return gB != kNone && ((bitB[v >> 6] >> (v & 63)) & 1); };
    mark("giants");
    // Main pass.  Each core-core edge not inside A or B is taken once:
    //   u in A: none; u in B: v in A; otherwise: v in A or B, or v < u.
    {
        std::atomic<uint64_t> next{0};
        const uint64_t blk = 2048;
        auto work = [&](uint64_t, uint64_t, int) {
            while (true) {
                uint64_t a = next.fetch_add(blk);
                if (a >= n) break;
                uint64_t b = std::min(n, a + blk);
                for (uint64_t u = a; u < b; ++u) {
                    if (!core[u] || inA((uint32_t)u)) continue;
                    const bool ub = inB((uint32_t)u);
                    const uint32_t* L = V + B[u];
                    uint32_t ru = uf_find(parent.get(), (uint32_t)u);   // kept current across the list
                    for (uint32_t i = 0, m = C[u]; i < m; ++i) {
                        const uint32_t v = L[i];
                        const bool va = inA(v);
                        if (!(ub ? va : (va || v < u || inB(v))) || !core[v]) continue;
                        const uint32_t rv = uf_find(parent.get(), v);
                        if (rv == ru) continue;                        // already joined: no link needed
                        uf_union(parent.get(), ru, rv);
                        ru = uf_find(parent.get(), ru);
                    }
                }
            }
        };
        if (T <= 1 || n < 4096) {
            work(0, n, 0);
        } else {
            std::vector<std::thread> th;
            for (int k = 0; k < T; ++k) th.emplace_back(work, 0, 0, k);
            for (auto& x : th) x.join();
        }
    }
    mark("union");
    // roots -> cluster numbers in increasing root (= minimum core) id
    std::vector<uint32_t> root(n ? n : 1);
    std::vector<uint64_t> part_cnt(T + 1, 0);
    uint64_t chunk = (n + T - 1) / std::max(T, 1);
    parallel_for(T, n, [&](uint64_t a, uint64_t b, int) {
        for (uint64_t p = a; p < b; ++p)
            if (core[p]) root[p] = uf_find(parent.get(), (uint32_t)p);
    });
    // prefix count of roots, chunked to match parallel_for's partition
    const bool serial = (T <= 1 || n < 4096);
    std::vector<uint32_t> rank_of(n ? n : 1);
    if (serial) {
        uint32_t k = 0;
        for (uint64_t p = 0; p < n; ++p)
            if (core[p] && root[p] == p) rank_of[p] = k++;
        part_cnt[0] = k;
    } else {
        std::vector<uint64_t> cnt(T, 0);
        parallel_for(T, n, [&](uint64_t a, uint64_t b, int k) {
            uint64_t c = 0;
            for (uint64_t p = a; p < b; ++p) c += (core[p] && root[p] == p);
            cnt[k] = c;
        });
        std::vector<uint64_t> pre(T + 1, 0);
        for (int k = 0; k < T; ++k) pre[k + 1] = pre[k] + cnt[k];
        parallel_for(T, n, [&](uint64_t a, uint64_t b, int k) {
            uint64_t r = pre[k];
            for (uint64_t p = a; p < b; ++p)
                if (core[p] && root[p] == p) rank_of[p] = (uint32_t)r++;
        });
        part_cnt[0] = pre[T];
    }
    (void)chunk;
    mark("roots+ranks");
    const uint32_t nclusters = (uint32_t)part_cnt[0];
    parallel_for(T, n, [&](uint64_t a, uint64_t b, int) {
        for (uint64_t p = a; p < b; ++p) {
            if (core[p]) {
                labels[p] = (int32_t)rank_of[root[p]];
            } else {
                int32_t best = -1;
                const uint32_t* L = V + B[p];
                for (uint32_t i = 0, m = C[p]; i < m; ++i) {
                    uint32_t v = L[i];
                    if (core[v]) {
                        int32_t c = (int32_t)rank_of[root[v]];
                        if (best < 0 || c < best) best = c;
                    }
                }
                labels[p] = best;
            }
        }
    });
    mark("labels");
    if (trace) fprintf(stderr, "[hdb trace] dbscan_par n=%llu threads=%d:%s\n", (unsigned long long)n, T, tlog.c_str());
    return nclusters;
}

}  // namespace

uint32_t dbscan_host(const hdb_table* t, uint32_t minpts, int n_threads, int32_t* labels, uint8_t* core_out) {
    std::vector<uint8_t> core_tmp;
    uint8_t* core = core_out;
    if (!core) {
        core_tmp.resize(t->n ? t->n : 1);
        core = core_tmp.data();
    }
    if (n_threads <= 1) return dbscan_seq(t, minpts, labels, core);
    return dbscan_par(t, minpts, n_threads, labels, core);
}

// Rows in id order, lists ascending; replaces the table's storage.
void canonicalize(hdb_table* t) {
    const uint64_t n = t->n;
    uint64_t* nb = (uint64_t*)malloc(8 * (n ? n : 1));
    uint32_t* nc = (uint32_t*)malloc(4 * (n ? n : 1));
    uint32_t* nv = (uint32_t*)malloc(4 * (t->npairs ? t->npairs : 1));
    if (!nb || !nc || !nv) {
        free(nb);
        free(nc);
        free(nv);
        fail(HDB_ENOMEM, "canonicalize: host allocation failed");
    }
    uint64_t acc = 0;
    for (uint64_t p = 0; p < n; ++p) {
        nb[p] = acc;
        nc[p] = t->count[p];
        acc += t->count[p];
    }
    const int T = resolve_threads(t->host_threads);
    parallel_for(T, n, [&](uint64_t a, uint64_t b, int) {
        for (uint64_t p = a; p < b; ++p) {
            memcpy(nv + nb[p], t->nbrs + t->begin[p], 4ull * nc[p]);
            std::sort(nv + nb[p], nv + nb[p] + nc[p]);
        }
    });
    if (t->pool) {
        t->pool->release(t->begin, t->cap_begin);
        t->pool->release(t->count, t->cap_count);
        t->pool->release(t->nbrs, t->cap_nbrs);
        t->pool.reset();
    } else if (t->malloced) {
        free(t->begin);
        free(t->count);
        free(t->nbrs);
    }
    t->begin = nb;
    t->count = nc;
    t->nbrs = nv;
    t->npairs = acc;
    t->malloced = true;
    // first_query / end_query are kept: a process shard stays a shard (hdb_dbscan rejects it)
}

}  // namespace hdb
