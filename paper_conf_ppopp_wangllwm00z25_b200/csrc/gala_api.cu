// gala_api.cu — host driver and C ABI of libgala.so (include/gala.h).
//
// The driver runs the multi-level loop of P:109 on the device: per level it
// initialises singletons (a1), iterates phase 1 (Alg. 1) until the
// exact numerator gain drops below T (a2-a7; one 64-byte D2H read per
// iteration carries the device's convergence decision), then relabels (a8)
// and coarsens (a9).  Every arithmetic step runs in the kernels of
// k_phase1.cuh / k_phase2.cuh; this file only sizes launches, owns memory and
// keeps statistics.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <map>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "gala.h"
#include "common.cuh"
#include "k_phase1.cuh"
#include "k_decide.cuh"
#include "k_phase2.cuh"
#include "comm.cuh"
#include "k_dist.cuh"
#include "fabric.cuh"
#include "k_nmi.cuh"
#ifndef GALA_APPLY_AGG
#define GALA_APPLY_AGG 1   // k_apply: warp-combined Sigma_tot / size atomics (d(v) < 2^32)
#endif

#define GALA_VERSION "gala-b200 0.1 (sm_100a)"

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;
static gala_status set_err(gala_status st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return st;
}
struct GalaError {
    gala_status st;
};
#define CK(call)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess) {                                                                   \
            set_err(e_ == cudaErrorMemoryAllocation ? GALA_E_NOMEM : GALA_E_CUDA, "%s:%d %s: %s", \
                    __FILE__, __LINE__, #call, cudaGetErrorString(e_));                           \
            throw GalaError{e_ == cudaErrorMemoryAllocation ? GALA_E_NOMEM : GALA_E_CUDA};        \
        }                                                                                          \
    } while (0)
// every kernel launch site is followed by CKL(), which also counts the launch
static thread_local long long g_launches = 0;
#define CKL()                       \
    do {                            \
        ++g_launches;               \
        CK(cudaGetLastError());     \
    } while (0)

// ------------------------------------------------------------------ kernel classes
enum KClass {
    KC_PRUNE = 0, KC_DEC_SMALL, KC_DEC_WARP, KC_DEC_WARP2, KC_DEC_BLOCK, KC_DEC_HUB,
    KC_APPLY, KC_DP, KC_REDUCE, KC_INIT, KC_PHASE2, KC_DEC_SINGLE, KC_XCHG, KC_COUNT
};
static const char* kc_names[KC_COUNT] = {"prune_bin", "decide_small", "decide_warp", "decide_warp512",
                                         "decide_block", "decide_hub", "apply",
                                         "dp_update", "reduce", "level_init", "phase2",
                                         "decide_single", "exchange"};

struct TraceRec {
    int64_t v[16];
};

struct DevCSR {
    int64_t n = 0, nnz = 0;
    int64_t* rp = nullptr;
    int32_t* col = nullptr;
    int64_t* w = nullptr;     // nullptr = unit weights
    int32_t* row = nullptr;   // row (source vertex) of every entry, for edge-parallel passes
};

struct LevelStat {
    int64_t n, nnz, iters, maxdeg;
    int i128path;
    double ms_phase1, ms_phase2;
    int64_t edges_scanned, nominal_edges;
    double alg_bytes;   // algorithmic bytes of the level's phase-1 iterations
    double ms_iters;    // device time of the level's iterations (globaltimer, first reduce -> last reduce)
};

struct gala_graph_s {
    int device = 0;
    cudaStream_t stream = nullptr;
    struct DevCache* cache = nullptr;
    bool own_stream = false;
    int num_sms = 148;
    // level-0 graph
    DevCSR g0;
    int64_t n0 = 0, nnz0 = 0, W = 0, maxdeg0 = 0, maxw0 = 0;
    int64_t* d0 = nullptr;
    int64_t* s0 = nullptr;
    // options
    int opt_prune = 1, opt_prune_check = 0, opt_trace = 0, opt_check = 0, opt_timing = 0, opt_max_iters = 0;
    int opt_delta_den = 2;   // adaptive d' update: delta iff moved row entries <= nnz / opt_delta_den
    int opt_delta = 2, opt_force_i128 = 0, opt_force_wide = 0, opt_cuda_graph = 1, opt_log_cap = 4096, opt_singleton = 1, opt_verbose = 0, opt_agg_big_chunk = 1,
        opt_agg_chunk = AGG_CH, opt_agg_scap = 8192;
    long long opt_agg_big_ent = 32768;   // communities with more entries take the chunked big path (any table size)
    int opt_block_split = 1024;
    int opt_agg_bound = 1;
    int opt_agg_dense = 1;
    int opt_l2_window = 0;   // persisting L2 access-policy window on C (A/B option)
    int opt_table_mode = 0;  // block bin's hash table: 0 hierarchical (§4.2), 1 global-only, 2 unified (ablation)
    double tbl[4] = {0, 0, 0, 0};   // last run: H0 / H1 accesses, H0 / H1 distinct keys of the block bin
    int opt_agg_spill = 1;   // phase 2: class D (one block, shared H0 spilling to global H1) for short segments
    int opt_bin_packed = 1;  // DM_W64 levels: packed argmax keys for the short-row bins where they fit   // phase 2: dense k x k accumulation when k <= AGG_DENSE_K and nnz >= 4 k^2
    bool rows_distinct0 = false;   // level-0 rows strictly increasing (no duplicate entries)
    bool self0 = true;             // level 0 has a self-loop (s0 not all zero)
    bool ckey_ok = false;          // level 0 may use the per-entry neighbour-community array (ckey)
    int opt_ckey = 0;
    int bins[NBINS - 1] = {4, 8, 16, 32, 128, 512, 16384};
    int hub_smem_slots = 8192;
    int opt_hub_cluster = 1;
    // results
    bool has_result = false;
    int64_t k = 0, p = 1, q = 1;
    i128 N = 0;
    int32_t* lab = nullptr;   // device, n0
    std::vector<TraceRec> trace;
    std::vector<std::vector<int32_t>> trace_labels;
    std::vector<LevelStat> levels;
    double kc_ms[KC_COUNT] = {0};
    double kc_bytes[KC_COUNT] = {0};
    int64_t kc_launches[KC_COUNT] = {0};
    double run_ms = 0;
    int64_t dp_mismatch = 0;
    long long launches = 0;   // kernels launched by the last gala_run
    int check_mismatch = 0;   // check mode: final N on G0 differs from the last level's N
    // multi-GPU (one process per GPU)
    struct DistInfo* di = nullptr;
    bool fab_host_bar = false;   // = di->host_bar (fabric barriers on the host: loopback ranks on one device)
    int64_t k_final = -1;        // communities of the last completed run (labels 0..k-1)
    int sync_mode = 0;
    std::vector<long long> dbounds0;   // level-0 owned ranges of all ranks
    struct Work* wk = nullptr;   // persistent run workspace (sized for level 0, reused by every run)
    int64_t cur_n = 0;           // vertex count of the level being iterated (trace label snapshots)
    // side streams of the decide fork: the bins' decide kernels are independent (disjoint
    // vertices, per-bin cursors and tables), so they run as parallel graph branches
    int opt_concurrent = 0;
    cudaStream_t side[4] = {nullptr, nullptr, nullptr, nullptr};
    cudaEvent_t ev_fork = nullptr, ev_join[4] = {nullptr, nullptr, nullptr, nullptr};
};

// Fork/join of independent launches onto the side streams.  Inside a stream
// capture the event record/wait pairs become graph edges (parallel branches of
// the conditional body); outside they are plain cross-stream dependencies.
// Per-kernel timing (events on the main stream) keeps everything serial.
struct Fork {
    gala_graph_s* g;
    bool on;
    int used = 0;
    explicit Fork(gala_graph_s* gg) : g(gg), on(gg->opt_concurrent && !gg->opt_timing) {
        if (!on) return;
        if (!g->ev_fork) {
            CK(cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming));
            for (int i = 0; i < 4; ++i) {
                CK(cudaStreamCreateWithFlags(&g->side[i], cudaStreamNonBlocking));
                CK(cudaEventCreateWithFlags(&g->ev_join[i], cudaEventDisableTiming));
            }
        }
        CK(cudaEventRecord(g->ev_fork, g->stream));
    }
    // stream for branch i (0..3); the main stream when forking is off
    cudaStream_t branch(int i) {
        if (!on) return g->stream;
        CK(cudaStreamWaitEvent(g->side[i], g->ev_fork, 0));
        used |= 1 << i;
        return g->side[i];
    }
    void join() {
        if (!on) return;
        for (int i = 0; i < 4; ++i)
            if (used & (1 << i)) {
                CK(cudaEventRecord(g->ev_join[i], g->side[i]));
                CK(cudaStreamWaitEvent(g->stream, g->ev_join[i], 0));
            }
        used = 0;
    }
    ~Fork() { join(); }
};

// ------------------------------------------------------------------ memory
// All device memory of a handle comes from its own stream-ordered pool (release
// threshold "keep everything") through a size-class cache: freed blocks are
// kept per handle and handed back to the next request of (nearly) the same
// size.  A run on the same graph repeats its allocation sequence, so from the
// second run on no allocation reaches the pool -- pool reuse alone would still
// remap physical pages to new virtual ranges (tens of ms per GB on big levels).
// Every user of a handle's memory is ordered on the handle's stream, which makes
// reuse without events safe.  The active cache is set per API call (PoolScope).
// User allocator hook (gala_set_allocator): when set, every device block the
// library allocates from then on comes from alloc_fn and goes back through free_fn (Python routes
// it to torch's caching allocator).  Each block remembers which allocator made it.
struct UserAlloc {
    gala_alloc_fn alloc = nullptr;
    gala_free_fn free = nullptr;
    void* ctx = nullptr;
};
static std::mutex g_ualloc_mu;
static UserAlloc g_ualloc;
static UserAlloc current_ualloc() {
    std::lock_guard<std::mutex> lk(g_ualloc_mu);
    return g_ualloc;
}
static int current_device() {
    int d = 0;
    cudaGetDevice(&d);
    return d;
}
struct BlockInfo {
    size_t bytes;
    UserAlloc ua;   // ua.alloc == nullptr: the stream-ordered pool / cudaMallocAsync
};
static void* user_alloc(const UserAlloc& ua, size_t bytes, cudaStream_t st) {
    void* p = ua.alloc(bytes, current_device(), (uintptr_t)st, ua.ctx);
    if (!p) {
        set_err(GALA_E_NOMEM, "user allocator returned NULL for %zu bytes", bytes);
        throw GalaError{GALA_E_NOMEM};
    }
    return p;
}

struct DevCache {
    cudaMemPool_t pool = nullptr;
    std::multimap<size_t, void*> freeb;        // cached free blocks by size
    std::unordered_map<void*, BlockInfo> sz;   // every block this cache handed out
    static size_t round(size_t b) {
        if (b <= 4096) return (b + 255) & ~(size_t)255;
        if (b < ((size_t)2 << 20)) { size_t r = 8192; while (r < b) r <<= 1; return r; }
        return (b + ((size_t)2 << 20) - 1) & ~(((size_t)2 << 20) - 1);
    }
    void* get(size_t bytes, cudaStream_t st) {
        const size_t r = round(bytes);
        const UserAlloc ua = current_ualloc();
        auto it = freeb.lower_bound(r);
        // reuse only blocks of the allocator now in effect
        for (; it != freeb.end() && it->first <= r + r / 4; ++it)
            if (sz[it->second].ua.alloc == ua.alloc && sz[it->second].ua.ctx == ua.ctx) {
                void* p = it->second;
                freeb.erase(it);
                return p;
            }
        void* p = nullptr;
        if (ua.alloc) {
            p = user_alloc(ua, r, st);
        } else {
            cudaError_t e = cudaMallocFromPoolAsync(&p, r, pool, st);
            if (e == cudaErrorMemoryAllocation) {
                // first the largest cached blocks back to the pool (stream-ordered: the pool reuses
                // their physical pages for this request, nothing is unmapped), then -- only if that
                // is not enough -- every cached block and the pool's unused reserve
                cudaGetLastError();
                size_t freed = 0;
                while (!freeb.empty() && freed < 2 * r) {
                    auto last = std::prev(freeb.end());
                    release(last->second, sz[last->second], st);
                    freed += last->first;
                    sz.erase(last->second);
                    freeb.erase(last);
                }
                e = cudaMallocFromPoolAsync(&p, r, pool, st);
                if (e == cudaErrorMemoryAllocation) {
                    cudaGetLastError();
                    trim(st);
                    cudaStreamSynchronize(st);
                    cudaMemPoolTrimTo(pool, 0);
                    e = cudaMallocFromPoolAsync(&p, r, pool, st);
                }
            }
            CK(e);
        }
        sz[p] = BlockInfo{r, ua};
        return p;
    }
    bool put(void* p) {
        auto it = sz.find(p);
        if (it == sz.end()) return false;
        freeb.emplace(it->second.bytes, p);
        return true;
    }
    static void release(void* p, const BlockInfo& b, cudaStream_t st) {
        if (b.ua.free) b.ua.free(p, b.bytes, current_device(), (uintptr_t)st, b.ua.ctx);
        else cudaFreeAsync(p, st);
    }
    void trim(cudaStream_t st) {
        for (auto& kv : freeb) {
            release(kv.second, sz[kv.second], st);
            sz.erase(kv.second);
        }
        freeb.clear();
    }
};
static thread_local DevCache* g_cache = nullptr;
// One retired cache per device: gala_graph_free parks its (idle, synchronised) pool and free
// blocks here and the next handle on that device adopts them, so repeated
// create/run/free cycles (e2e) do not map fresh physical pages each time.
static std::mutex g_stash_mu;
static std::map<int, DevCache*> g_stash;

// Process-wide stash of the small pinned host buffers of a run workspace (device log and carry
// mirrors): cudaMallocHost / cudaFreeHost cost milliseconds and synchronise the device, once per
// handle otherwise (the e2e create -> run -> free cycle).
static std::mutex g_pin_mu;
static std::multimap<size_t, void*> g_pin;
static void* pin_get(size_t n) {
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        auto it = g_pin.find(n);
        if (it != g_pin.end()) { void* p = it->second; g_pin.erase(it); return p; }
    }
    void* p = nullptr;
    if (cudaMallocHost(&p, n) != cudaSuccess) return nullptr;
    return p;
}
static void pin_put(void* p, size_t n) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(g_pin_mu);
    g_pin.emplace(n, p);
}
static bool cache_has_user_blocks(const DevCache* c) {
    for (auto& kv : c->sz)
        if (kv.second.ua.alloc) return true;
    return false;
}
struct PoolScope {
    DevCache* prev;
    explicit PoolScope(DevCache* c) : prev(g_cache) { g_cache = c; }
    ~PoolScope() { g_cache = prev; }
};
// blocks allocated outside any handle's cache by the user allocator (size + allocator kept for free)
static std::mutex g_loose_mu;
static std::unordered_map<void*, BlockInfo> g_loose;
template <typename T>
static T* dalloc(size_t count, cudaStream_t st) {
    if (count == 0) count = 1;
    if (g_cache) return static_cast<T*>(g_cache->get(count * sizeof(T), st));
    void* p = nullptr;
    const UserAlloc ua = current_ualloc();
    if (ua.alloc) {
        p = user_alloc(ua, count * sizeof(T), st);
        std::lock_guard<std::mutex> lk(g_loose_mu);
        g_loose[p] = BlockInfo{count * sizeof(T), ua};
        return static_cast<T*>(p);
    }
    CK(cudaMallocAsync(&p, count * sizeof(T), st));
    return static_cast<T*>(p);
}
template <typename T>
static void dfree(T*& p, cudaStream_t st) {
    if (p && !(g_cache && g_cache->put(p))) {
        BlockInfo b{0, UserAlloc{}};
        bool loose = false;
        {
            std::lock_guard<std::mutex> lk(g_loose_mu);
            auto it = g_loose.find((void*)p);
            if (it != g_loose.end()) { b = it->second; g_loose.erase(it); loose = true; }
        }
        if (loose) DevCache::release((void*)p, b, st);
        else cudaFreeAsync(p, st);
    }
    p = nullptr;
}

static int grid_for(long long n, int bt, int cap) {
    long long g = (n + bt - 1) / bt;
    if (g < 1) g = 1;
    if (g > cap) g = cap;
    return (int)g;
}

// exclusive scan of int64 in[0..n) into out[0..n] (out[n] = total)
static void scan_excl(const long long* in, long long* out, long long n, cudaStream_t st) {
    long long nt = (n + SCAN_TILE - 1) / SCAN_TILE;
    if (nt < 1) nt = 1;
    long long* sums = dalloc<long long>(nt + 1, st);
    k_scan_tiles<<<(unsigned)nt, SCAN_BT, 0, st>>>(in, n, sums);
    CKL();
    k_scan_sums<<<1, SCAN_BT, 0, st>>>(sums, nt);
    CKL();
    k_scan_apply<<<(unsigned)nt, SCAN_BT, 0, st>>>(in, n, sums, out, nt);
    CKL();
    dfree(sums, st);
}

// ------------------------------------------------------------------ timing
struct Timer {
    gala_graph_s* g;
    std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> pending;
    std::vector<cudaEvent_t> pool;
    explicit Timer(gala_graph_s* gg) : g(gg) {}
    cudaEvent_t get() {
        if (!pool.empty()) { cudaEvent_t e = pool.back(); pool.pop_back(); return e; }
        cudaEvent_t e;
        CK(cudaEventCreate(&e));
        return e;
    }
    cudaEvent_t begin() {
        if (!g->opt_timing) return nullptr;
        cudaEvent_t e = get();
        CK(cudaEventRecord(e, g->stream));
        return e;
    }
    void end(int kc, cudaEvent_t b) {
        g->kc_launches[kc]++;
        if (!g->opt_timing) return;
        cudaEvent_t e = get();
        CK(cudaEventRecord(e, g->stream));
        pending.push_back({kc, {b, e}});
    }
    void resolve() {   // call after a stream sync
        for (auto& x : pending) {
            float ms = 0;
            CK(cudaEventElapsedTime(&ms, x.second.first, x.second.second));
            g->kc_ms[x.first] += ms;
            pool.push_back(x.second.first);
            pool.push_back(x.second.second);
        }
        pending.clear();
    }
    ~Timer() {
        for (auto& x : pending) { cudaEventDestroy(x.second.first); cudaEventDestroy(x.second.second); }
        for (auto e : pool) cudaEventDestroy(e);
    }
};

// ------------------------------------------------------------------ gamma, thresholds
static int64_t gcd64(int64_t a, int64_t b) {
    while (b) { int64_t t = a % b; a = b; b = t; }
    return a;
}
static void gamma_to_pq(double gamma, int64_t* p, int64_t* q) {
    int64_t pp = (int64_t)(gamma * 65536.0 + 0.5), qq = 65536;
    int64_t g = gcd64(pp, qq);
    if (g == 0) g = 1;
    *p = pp / g;
    *q = qq / g;
}

// ------------------------------------------------------------------ workspace of a run
struct Work {
    cudaStream_t st;
    int64_t ncap, nnzcap;
    long long icap = 0;   // capacity of the delta-update item arrays (light items from the front, others from the back)
    int64_t qcap = 0;   // queue stride (records per bin pair): n on one GPU, the largest owned range so far with several
    int32_t *rmflag = nullptr, *smflag = nullptr, *chg = nullptr;   // SM / RM movement history (prune 2-4)
    int32_t *C = nullptr, *size = nullptr, *stamp = nullptr, *mv_v = nullptr, *mv_old = nullptr, *mv_chunk = nullptr, *nextC = nullptr;
    QRec* queues = nullptr;
    int32_t* ckey = nullptr;   // level-0 per-entry neighbour community
    int2* cst = nullptr;       // (C[v], stamp[v]) pairs: one 8-byte gather per entry in k_dp_delta
    int64_t *Sig = nullptr, *d = nullptr, *s = nullptr, *dp = nullptr;
    bool s_zero = false;   // this level has no self-loops: k_reduce skips s (level 0 of a loop-free graph)
    const int64_t* s_live() const { return s_zero ? nullptr : s; }
    IterCounters* ctr = nullptr;
    Carry* carry = nullptr;
    IterLog* log = nullptr;
    int log_cap = 4096;
    long long *part_dc = nullptr, *part_min = nullptr;
    i128* part_s2 = nullptr;
    int* gkeys = nullptr;
    ull* gvals = nullptr;
    int* glist = nullptr;
    long long gcap = 0;
    int gblocks = 0;          // max over modes (spill-table count)
    int gblocks_m[3] = {0, 0, 0};
    // hub tables (k_hub_*), sized per level for the rows longer than the block bin
    bool hub_on = false;
    bool hub_cluster = false;   // this level's hubs take the cluster kernel (k_decide_cluster)
    HubWork hw = {};
    long long hub_ncap = 0, hub_tcap = 0, hub_lcap = 0, hub_pcap = 0;
    ull* hub_size = nullptr;
    IterLog* h_log = nullptr;
    Carry* h_carry = nullptr;
    int reduce_grid = 0;
    int smem_cap = 0;
    cudaEvent_t ev[5] = {nullptr, nullptr, nullptr, nullptr, nullptr};
    void release() {
        for (auto& e : ev) if (e) { cudaEventDestroy(e); e = nullptr; }
        dfree(C, st); dfree(size, st); dfree(stamp, st); dfree(mv_v, st); dfree(mv_old, st); dfree(mv_chunk, st);
        dfree(rmflag, st); dfree(smflag, st); dfree(chg, st); dfree(nextC, st);
        dfree(queues, st); dfree(ckey, st); dfree(cst, st); dfree(Sig, st); dfree(d, st); dfree(s, st); dfree(dp, st); dfree(ctr, st);
        dfree(carry, st); dfree(log, st); dfree(part_dc, st); dfree(part_min, st); dfree(part_s2, st);
        dfree(gkeys, st); dfree(gvals, st); dfree(glist, st);
        dfree(hw.keys, st); dfree(hw.vals, st); dfree(hw.list, st); dfree(hw.pref, st); dfree(hw.toff, st);
        dfree(hw.loff, st); dfree(hw.cnt, st); dfree(hub_size, st); dfree(hw.spref, st); dfree(hw.own, st);
        char* part = static_cast<char*>(hw.part);
        dfree(part, st);
        hw.part = nullptr;
        hub_ncap = hub_tcap = hub_lcap = hub_pcap = 0;
        pin_put(h_log, sizeof(IterLog) * (size_t)log_cap);
        pin_put(h_carry, sizeof(Carry));
        h_log = nullptr;
        h_carry = nullptr;
    }
};

#ifndef GALA_BLOCK_BT
#define GALA_BLOCK_BT 512
#endif
#ifndef GALA_BLOCK_E
#define GALA_BLOCK_E 2
#endif
#define BLOCK_BT GALA_BLOCK_BT
#define BLOCK_E GALA_BLOCK_E
// short-row class of the block bin (rows <= opt_block_split): 256 threads, 4 entries each
#define BLOCK_LO_BT 256
#define BLOCK_LO_E 4

// ------------------------------------------------------------------ launch helpers
// the per-entry neighbour-community array is used on level 0 of single-GPU runs
static bool use_ckey(const gala_graph_s* g, const Work& wk, const DevCSR& G) {
    return g->opt_ckey && g->ckey_ok && wk.ckey && !g->di && G.col == g->g0.col;
}

// pruning strategy state of a run; the SM / RM history arrays are allocated on first use
static PruneState prune_state(gala_graph_s* g, Work& wk) {
    PruneState ps;
    ps.mode = g->opt_prune;
    ps.instr = g->opt_prune_check;
    if ((ps.mode == 3 || ps.mode == 4) && !wk.rmflag) wk.rmflag = dalloc<int32_t>(wk.ncap, g->stream);
    if (ps.mode == 2 && !wk.smflag) {
        wk.smflag = dalloc<int32_t>(wk.ncap, g->stream);
        wk.chg = dalloc<int32_t>(wk.ncap, g->stream);
    }
    ps.rmflag = (ps.mode == 3 || ps.mode == 4) ? wk.rmflag : nullptr;
    ps.smflag = ps.mode == 2 ? wk.smflag : nullptr;
    ps.chg = ps.mode == 2 ? wk.chg : nullptr;
    return ps;
}

template <int GW, int MAXDEG, int M>
static void set_warp_smem() {
    CK(cudaFuncSetAttribute(k_decide_warp<GW, MAXDEG, M, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)WarpSmem<GW, MAXDEG, M>::bytes));
    CK(cudaFuncSetAttribute(k_decide_warp<GW, MAXDEG, M, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)WarpSmem<GW, MAXDEG, M>::bytes));
}
template <int M>
static size_t block_smem_bytes(int cap) { return (size_t)cap * (sizeof(typename ModeT<M>::VT) + sizeof(int)); }

// multi-block hub path (bin BIN_HUB), only on levels that have such rows
template <int M, bool UNIT>
static void launch_hub(gala_graph_s* g, Work& wk, const DecideArgs& a, typename ModeT<M>::ST qW,
                       typename ModeT<M>::ST p, Timer& tm, cudaStream_t st) {
    if (!wk.hub_on) return;
    const QView q = qview(wk.queues, wk.qcap, BIN_HUB);
    cudaEvent_t e = tm.begin();
    if constexpr (M != DM_W128) {
        if (wk.hub_cluster) {   // tables in the distributed shared memory of a thread-block cluster
            const int grid = std::max(g->num_sms / CL_CS, 1) * CL_CS;
            k_decide_cluster<M, UNIT><<<grid, CL_BT, CL_SLOTS * sizeof(ull), st>>>(q, a, qW, p);
            CKL();
            tm.end(KC_DEC_HUB, e);
            return;
        }
    }
    k_hub_prep<<<1, 1024, 0, st>>>(q, wk.ctr, wk.hw);
    CKL();
    k_hub_agg<M, UNIT><<<g->num_sms * 8, HUB_BT, 0, st>>>(q, a, wk.hw);
    CKL();
    k_hub_prep2<<<1, 1024, 0, st>>>(wk.ctr, wk.hw);
    CKL();
    k_hub_eval<M, UNIT><<<g->num_sms * 4, HUB_EVAL_BT, 0, st>>>(q, a, wk.hw, qW, p);
    CKL();
    k_hub_final<M, UNIT><<<g->num_sms, 256, 0, st>>>(q, a, wk.hw, qW, p);
    CKL();
    tm.end(KC_DEC_HUB, e);
}

// DM_FAST's packed (score, -c) argmax keys need max(p,q) W d(v) 2^idbits < 2^62 for the vertices
// a kernel evaluates -- not for the level's largest degree.  On a unit-weight level d(v) is the row
// length, so the bins of rows up to `rowmax` can use packed keys (one 64-bit max per reduction
// step) even when the level's hubs need DM_W64's (score, c) pairs.  Same integers either way.
static bool packed_ok(const gala_graph_s* g, int idbits, int64_t rowmax) {
    return (long double)std::max(g->p, g->q) * (long double)g->W * (long double)std::max<int64_t>(rowmax, 1) *
               (long double)((int64_t)1 << idbits) < 0x1p62L;
}

template <int M, bool UNIT>
static void launch_single(gala_graph_s* g, Work& wk, const DecideArgs& a, typename ModeT<M>::ST qW,
                          typename ModeT<M>::ST p, Timer& tm, int64_t maxdeg) {
    const long long qs = wk.qcap;
    const int grid = g->num_sms * 8;
    cudaStream_t st = g->stream;
    Fork fk(g);
    // rows <= bins[BIN_WARP2] with packed argmax keys where they fit (packed_ok)
    bool fast = false;
    if constexpr (M == DM_W64 && UNIT)
        fast = g->opt_bin_packed && g->opt_force_wide != 1 && packed_ok(g, a.idbits, std::min<int64_t>(maxdeg, g->bins[BIN_WARP2]));
    cudaEvent_t e = tm.begin();
    if (fast) k_decide_single_small<DM_FAST, UNIT><<<grid, 256, 0, st>>>(wk.queues, qs, a, qW, p);
    else k_decide_single_small<M, UNIT><<<grid, 256, 0, st>>>(wk.queues, qs, a, qW, p);
    CKL();
    tm.end(KC_DEC_SINGLE, e);
    for (int b = BIN_WARP; b <= BIN_BLOCK; ++b) {
        if (maxdeg <= g->bins[b - 1]) break;
        e = tm.begin();
        if (fast && b <= BIN_WARP2)
            k_decide_single<DM_FAST, UNIT><<<grid, 256, 0, fk.branch(b - BIN_WARP)>>>(qview(wk.queues, qs, b), b, a, qW, p);
        else k_decide_single<M, UNIT><<<grid, 256, 0, fk.branch(b - BIN_WARP)>>>(qview(wk.queues, qs, b), b, a, qW, p);
        CKL();
        tm.end(KC_DEC_SINGLE, e);
    }
    if (wk.hub_on) {   // singleton hubs: chunked argmax, no tables
        const QView q = qview(wk.queues, wk.qcap, BIN_HUB);
        cudaStream_t hs = fk.branch(3);
        e = tm.begin();
        k_hub_prep<<<1, 1024, 0, hs>>>(q, wk.ctr, wk.hw);
        CKL();
        k_hub_single_chunk<M, UNIT><<<g->num_sms * 8, HUB_BT, 0, hs>>>(q, a, wk.hw, qW, p);
        CKL();
        k_hub_single_final<M, UNIT><<<g->num_sms, 256, 0, hs>>>(q, a, wk.hw);
        CKL();
        tm.end(KC_DEC_HUB, e);
    }
}

// Dynamic shared-memory limits of the block kernels.  The limit is a per-function, process-wide
// attribute: it is only ever RAISED (under a lock, before any capture) to the largest arena a handle
// needs, so handles with different options (loopback ranks are threads) never see a limit below
// their own arena.  It is not simply set to the largest arena any option allows: a larger limit
// measurably slows the default configuration (orkut decide_block 8.6 -> 11.3 ms with a 16384-slot
// limit; the shared-memory carveout follows the limit, leaving less L1 for the gathers).
template <int M, bool UNIT>
static void block_attr_mode(int slots) {
    const int mx = (int)block_smem_bytes<M>(slots);
    CK(cudaFuncSetAttribute(k_decide_block<BLOCK_BT, BLOCK_E, M, UNIT>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
    CK(cudaFuncSetAttribute(k_decide_block<BLOCK_BT, BLOCK_E, M, UNIT, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
    CK(cudaFuncSetAttribute(k_decide_block<BLOCK_LO_BT, BLOCK_LO_E, M, UNIT, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
    CK(cudaFuncSetAttribute(k_decide_block<BLOCK_LO_BT, BLOCK_LO_E, M, UNIT, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, mx));
}
static void block_attrs_ensure(int slots) {
    static std::mutex mu;
    static std::map<int, int> cur;   // per device: slots the limits allow
    std::lock_guard<std::mutex> lk(mu);
    const int dev = current_device();
    if (cur[dev] >= slots) return;
    block_attr_mode<DM_FAST, true>(slots); block_attr_mode<DM_FAST, false>(slots);
    block_attr_mode<DM_W64, true>(slots); block_attr_mode<DM_W64, false>(slots);
    block_attr_mode<DM_W128, true>(slots); block_attr_mode<DM_W128, false>(slots);
    if (!cur.count(-1 - dev)) {   // cluster hub kernel: its fixed 128 KB per CTA
        const int cs = CL_SLOTS * (int)sizeof(ull);
        CK(cudaFuncSetAttribute(k_decide_cluster<DM_FAST, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, cs));
        CK(cudaFuncSetAttribute(k_decide_cluster<DM_FAST, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, cs));
        CK(cudaFuncSetAttribute(k_decide_cluster<DM_W64, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, cs));
        CK(cudaFuncSetAttribute(k_decide_cluster<DM_W64, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, cs));
        cur[-1 - dev] = 1;
    }
    cur[dev] = slots;
}
// the largest block arena this handle launches (the short-row class runs only when its arena is
// smaller than hub_smem_slots)
static int block_arena_slots(const gala_graph_s* g) { return g->hub_smem_slots; }

// grid of the short-row block kernel (rows <= opt_block_split): resident blocks per SM for its
// arena, computed once per (mode, unit, arena, class)
template <int M, bool UNIT>
static int block_lo_grid(gala_graph_s* g, int cap, bool all) {
    static std::map<std::pair<int, int>, int> memo;
    static std::mutex mu;
    const std::pair<int, int> key(cap, all ? 1 : 0);
    const void* f = all ? (const void*)k_decide_block<BLOCK_LO_BT, BLOCK_LO_E, M, UNIT, 0>
                        : (const void*)k_decide_block<BLOCK_LO_BT, BLOCK_LO_E, M, UNIT, 1>;
    const size_t sm = block_smem_bytes<M>(cap);
    std::lock_guard<std::mutex> lk(mu);
    auto it = memo.find(key);
    if (it != memo.end()) return g->num_sms * it->second;
    int b = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, f, BLOCK_LO_BT, sm));
    b = std::max(b, 1);
    memo[key] = b;
    return g->num_sms * b;
}

// every block-kernel attribute / grid the launches need, set up front: nothing of this may run
// while a level's iteration body is being captured into a CUDA graph
template <int M, bool UNIT>
static void block_setup(gala_graph_s* g) {
    block_attrs_ensure(block_arena_slots(g));
    int cap1 = 64;
    while (cap1 < 2 * std::max(g->opt_block_split, 1)) cap1 <<= 1;
    if (cap1 < g->hub_smem_slots) (void)block_lo_grid<M, UNIT>(g, cap1, false);   // the only case it launches
}

// the sub-warp and warp bins (rows <= bins[BIN_WARP2]); MS: mode of the sub-warp kernel (packed keys
// pay there: A/B on orkut decide_small 2.37 -> 2.16 ms), M: the warp kernels' (the packed variant of
// the 128-row warp kernel spills; measured 4.98 -> 5.34 ms)
template <int M, bool UNIT, int MS = M, int MW = M>
static void launch_short_bins(gala_graph_s* g, Work& wk, const DecideArgs& a, typename ModeT<M>::ST qW,
                              typename ModeT<M>::ST p, Timer& tm, int64_t maxdeg, Fork& fk) {
    const long long qs = wk.qcap;
    const int grid = g->num_sms * 8;
    cudaStream_t st = g->stream;
    cudaEvent_t e = tm.begin();
    k_decide_small<MS, UNIT><<<grid, 256, 0, st>>>(wk.queues, qs, a, qW, p);
    CKL();
    tm.end(KC_DEC_SMALL, e);
    e = tm.begin();
    k_decide_warp<32, 128, MW, UNIT><<<grid, 32 * WarpSmem<32, 128, MW>::WPB, WarpSmem<32, 128, MW>::bytes, fk.branch(2)>>>(
        qview(wk.queues, qs, BIN_WARP), BIN_WARP, a, qW, p);
    CKL();
    tm.end(KC_DEC_WARP, e);
    if (maxdeg > g->bins[BIN_WARP]) {
        e = tm.begin();
        k_decide_warp<32, 512, MW, UNIT><<<grid, 32 * WarpSmem<32, 512, MW>::WPB, WarpSmem<32, 512, MW>::bytes,
                                           fk.branch(3)>>>(qview(wk.queues, qs, BIN_WARP2), BIN_WARP2, a, qW, p);
        CKL();
        tm.end(KC_DEC_WARP2, e);
    }
}

template <int M, bool UNIT>
static void launch_decide(gala_graph_s* g, Work& wk, const DevCSR& G, typename ModeT<M>::ST qW,
                          typename ModeT<M>::ST p, Timer& tm, int64_t maxdeg, int idbits, bool single) {
    DecideArgs a;
    a.rp = G.rp; a.col = G.col; a.w = G.w; a.C = wk.C; a.Sig = wk.Sig; a.size = wk.size; a.d = wk.d;
    a.dp = wk.dp; a.nextC = wk.nextC; a.ctr = wk.ctr; a.check = g->opt_check;
    a.table_mode = g->opt_table_mode;
    a.nlev = G.n;
    a.ckey = use_ckey(g, wk, G) ? wk.ckey : nullptr;
    a.ckey_valid = &wk.carry->ckey_valid;
    a.idbits = idbits;
    a.idmask = (1LL << idbits) - 1;
    if (single) return launch_single<M, UNIT>(g, wk, a, qW, p, tm, maxdeg);
    const long long qs = wk.qcap;
    cudaStream_t st = g->stream;
    Fork fk(g);
    cudaEvent_t e;
    // the longest-running bins go first so they start on an idle machine
    if (maxdeg > g->bins[BIN_WARP2]) {
        const int smem_cap = g->hub_smem_slots;
        const int split = g->opt_block_split;
        int cap1 = 64;
        while (cap1 < 2 * split) cap1 <<= 1;
        if (split > 0 && cap1 < smem_cap && maxdeg > split) {
            // rows <= split: small blocks with an arena that never spills; longer rows: the full
            // arena (a level whose rows all fit the split keeps the single full-arena kernel:
            // measured faster there, lfr1m)
            const int grid1 = block_lo_grid<M, UNIT>(g, cap1, false);
            e = tm.begin();
            k_decide_block<BLOCK_LO_BT, BLOCK_LO_E, M, UNIT, 1><<<grid1, BLOCK_LO_BT, block_smem_bytes<M>(cap1),
                                                                 fk.branch(0)>>>(
                qview(wk.queues, qs, BIN_BLOCK), BIN_BLOCK, a, qW, p, cap1, wk.gkeys, wk.gvals, wk.glist, wk.gcap,
                split);
            CKL();
            tm.end(KC_DEC_BLOCK, e);
            {
                e = tm.begin();
                k_decide_block<BLOCK_BT, BLOCK_E, M, UNIT, 2><<<wk.gblocks_m[M], BLOCK_BT, block_smem_bytes<M>(smem_cap),
                                                               fk.branch(0)>>>(
                    qview(wk.queues, qs, BIN_BLOCK), BIN_BLOCK, a, qW, p, smem_cap, wk.gkeys, wk.gvals, wk.glist,
                    wk.gcap, split);
                CKL();
                tm.end(KC_DEC_BLOCK, e);
            }
        } else {
            e = tm.begin();
            k_decide_block<BLOCK_BT, BLOCK_E, M, UNIT><<<wk.gblocks_m[M], BLOCK_BT, block_smem_bytes<M>(smem_cap),
                                                         fk.branch(0)>>>(
                qview(wk.queues, qs, BIN_BLOCK), BIN_BLOCK, a, qW, p, smem_cap, wk.gkeys, wk.gvals, wk.glist, wk.gcap);
            CKL();
            tm.end(KC_DEC_BLOCK, e);
        }
    }
    launch_hub<M, UNIT>(g, wk, a, qW, p, tm, wk.hub_on ? fk.branch(1) : st);
    if constexpr (M == DM_W64 && UNIT) {   // short / mid rows may use packed argmax keys (packed_ok)
        if (g->opt_bin_packed && g->opt_force_wide != 1 && packed_ok(g, idbits, std::min<int64_t>(maxdeg, g->bins[BIN_WARP2])))
            return launch_short_bins<M, UNIT, DM_FAST, DM_FAST>(g, wk, a, qW, p, tm, maxdeg, fk);
        if (g->opt_bin_packed && g->opt_force_wide != 1 && packed_ok(g, idbits, std::min<int64_t>(maxdeg, g->bins[BIN_S32])))
            return launch_short_bins<M, UNIT, DM_FAST>(g, wk, a, qW, p, tm, maxdeg, fk);
    }
    launch_short_bins<M, UNIT>(g, wk, a, qW, p, tm, maxdeg, fk);
}

// Per level, before its iterations: per-block spill tables of the block bin
// (rows up to bins[BIN_BLOCK]) and the hub tables of the longer rows.
static void prepare_level_tables(gala_graph_s* g, Work& wk, const DevCSR& G, int64_t maxdeg) {
    cudaStream_t st = g->stream;
    const int64_t bmax = std::min<int64_t>(maxdeg, g->bins[BIN_BLOCK]);
    long long need = 64;
    while (need < 2 * bmax) need <<= 1;
    if (maxdeg > g->bins[BIN_WARP2] && need > wk.gcap) {
        dfree(wk.gkeys, st);
        dfree(wk.gvals, st);
        dfree(wk.glist, st);
        wk.gcap = need;
        wk.gkeys = dalloc<int>((size_t)wk.gblocks * wk.gcap, st);
        wk.gvals = dalloc<ull>((size_t)wk.gblocks * wk.gcap, st);
        wk.glist = dalloc<int>((size_t)wk.gblocks * wk.gcap, st);
        CK(cudaMemsetAsync(wk.gkeys, 0xff, sizeof(int) * (size_t)wk.gblocks * wk.gcap, st));
        CK(cudaMemsetAsync(wk.gvals, 0, sizeof(ull) * (size_t)wk.gblocks * wk.gcap, st));
    }
    wk.hub_on = maxdeg > g->bins[BIN_BLOCK];
    {   // every hub's table fits the cluster's distributed shared memory (load <= 1/2)
        long long need = 64LL * CL_CS;
        while (need < 2 * std::min<long long>(maxdeg, G.n)) need <<= 1;
        // (32-bit packed sums: launched only in the modes with 32-bit aggregates, d(v) < 2^32)
        wk.hub_cluster = wk.hub_on && g->opt_hub_cluster && need <= (long long)CL_CS * CL_SLOTS;
    }
    if (!wk.hub_on) return;
    if (!wk.hub_size) wk.hub_size = dalloc<ull>(3, st);
    CK(cudaMemsetAsync(wk.hub_size, 0, sizeof(ull) * 3, st));
    k_hub_size<<<grid_for(G.n, 256, g->num_sms * 8), 256, 0, st>>>(G.n, G.rp, g->bins[BIN_BLOCK], G.n, wk.hub_size);
    CKL();
    ull hs[3];
    CK(cudaMemcpyAsync(hs, wk.hub_size, sizeof(hs), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const long long nh = (long long)hs[0] + 1, tc = std::max<long long>((long long)hs[1], 1),
                    lc = std::max<long long>((long long)hs[2], 1);
    HubWork& h = wk.hw;
    if (nh > wk.hub_ncap) {
        dfree(h.pref, st); dfree(h.toff, st); dfree(h.loff, st); dfree(h.cnt, st); dfree(h.spref, st);
        dfree(h.own, st);
        h.pref = dalloc<long long>(nh, st);
        h.toff = dalloc<long long>(nh, st);
        h.loff = dalloc<long long>(nh, st);
        h.spref = dalloc<long long>(nh, st);
        h.cnt = dalloc<int>(nh, st);
        h.own = dalloc<long long>(nh, st);
        wk.hub_ncap = nh;
    }
    const long long np = lc / HUB_CH + nh + 1;   // evaluation slices (HUB_EV) or singleton chunks (HUB_CH)
    if (np > wk.hub_pcap) {
        char* part = static_cast<char*>(h.part);
        dfree(part, st);
        h.part = dalloc<char>((size_t)np * 32, st);
        wk.hub_pcap = np;
    }
    static_assert(sizeof(Arg<i128, false>) <= 32, "partial argmax record");
    if (tc > wk.hub_tcap) {
        dfree(h.keys, st); dfree(h.vals, st);
        h.keys = dalloc<int>(tc, st);
        h.vals = dalloc<ull>(tc, st);
        wk.hub_tcap = tc;
    }
    if (lc > wk.hub_lcap) {
        dfree(h.list, st);
        h.list = dalloc<int>(lc, st);
        wk.hub_lcap = lc;
    }
    // tables start empty on every level (evaluation keeps them empty afterwards)
    CK(cudaMemsetAsync(h.keys, 0xff, sizeof(int) * tc, st));
    CK(cudaMemsetAsync(h.vals, 0, sizeof(ull) * tc, st));
    CK(cudaMemsetAsync(h.cnt, 0, sizeof(int) * nh, st));
    CK(cudaMemsetAsync(h.own, 0, sizeof(long long) * nh, st));
    h.nlev = G.n;
}

// one phase-1 iteration (Alg. 1 lines 3-13) + its device log record
template <int M, bool UNIT>
static void issue_iteration(gala_graph_s* g, Work& wk, const DevCSR& G, typename ModeT<M>::ST qW,
                            typename ModeT<M>::ST p, i128 qW128, i128 T, Timer& tm, int64_t maxdeg, int idbits,
                            unsigned long long cond, bool single) {
    cudaStream_t st = g->stream;
    const int n = (int)G.n;
    const int big = g->num_sms * 8;
    cudaEvent_t e = tm.begin();
    // the counters were cleared by the previous iteration's reduce (or the level start)
    BinThresholds th;
    for (int i = 0; i < NBINS - 1; ++i) th.t[i] = g->bins[i];
    const PruneState ps = prune_state(g, wk);
    k_prune_bin<typename ModeT<M>::ST><<<grid_for((n + PB_IPT - 1) / PB_IPT, PB_BT, big), PB_BT, 0, st>>>(
        0, n, G.rp, wk.d, wk.dp, wk.C, wk.Sig, wk.size, ps, qW, p, wk.carry, wk.ctr, wk.queues, wk.qcap, th);
    CKL();
    tm.end(KC_PRUNE, e);
    launch_decide<M, UNIT>(g, wk, G, qW, p, tm, maxdeg, idbits, single);
    e = tm.begin();
    k_apply<<<grid_for(n, AP_BT, big), AP_BT, 0, st>>>(wk.ctr, wk.queues, wk.qcap, wk.nextC, wk.C, wk.Sig, wk.size,
                                                       wk.dp, wk.stamp, wk.cst, wk.carry, wk.mv_v, wk.mv_old, wk.mv_chunk, ps, wk.icap,
                                                       GALA_APPLY_AGG && g->W < ((int64_t)1 << 32) ? 1 : 0);
    CKL();
    tm.end(KC_APPLY, e);
    e = tm.begin();
    const bool ck = use_ckey(g, wk, G);
    k_dp_delta<UNIT><<<big, 256, 0, st>>>(wk.ctr, G.rp, G.col, G.w, wk.C, wk.cst, wk.mv_v, wk.mv_old, wk.mv_chunk, wk.stamp, wk.dp,
                                          wk.carry, G.nnz, g->opt_delta, 1, g->opt_delta_den, ck ? wk.ckey : nullptr,
                                          nullptr, ps.rmflag, n, wk.icap);
    CKL();
    k_dp_full<UNIT><<<grid_for((G.nnz + 127) / 128 * 32, 256, big), 256, 0, st>>>(wk.ctr, G.nnz, G.row, G.col, G.w,
                                                                                 wk.C, wk.dp, g->opt_delta, 1, g->opt_delta_den,
                                                                                 ck ? wk.ckey : nullptr, &wk.carry->ckey_valid,
                                                                                 ps.rmflag, wk.stamp, wk.carry);
    CKL();
    if (ps.mode == 2 && G.nnz) {   // SM: mark rows next to a community that changed
        k_sm_flags<<<grid_for(G.nnz, 256, big * 4), 256, 0, st>>>(G.nnz, G.row, G.col, wk.C, ps, wk.carry);
        CKL();
    }
    tm.end(KC_DP, e);
    e = tm.begin();
    k_reduce<256><<<wk.reduce_grid, 256, 0, st>>>(n, 0, n, wk.dp, wk.s_live(), wk.Sig, wk.part_dc, wk.part_s2, wk.part_min, wk.ctr,
                                                  wk.carry, (long long)(qW128 >> 64), (ull)qW128, (long long)p,
                                                  (long long)(T >> 64), (ull)T, 1, wk.log, wk.log_cap, g->opt_max_iters,
                                                  cond);
    CKL();
    tm.end(KC_REDUCE, e);
}

// Phase 1 of one level to convergence.  Graph mode: the iteration body is
// captured once into the body of a conditional WHILE node whose condition the
// iteration's last kernel sets on the device (no host round trip per iteration).
// Stepwise mode (trace labels, per-kernel timing, or cuda_graph=0): one host loop
// trip per iteration.  Both issue the identical kernels.  `issue(cond, single)`
// enqueues one iteration (single: the level's first, singleton fast path); the
// single-GPU and the multi-GPU (fabric) drivers share this loop.
struct NoHook {
    void operator()() const {}
};
template <typename Issue, typename PreLaunch = NoHook>
static void level_loop(gala_graph_s* g, Work& wk, std::vector<IterLog>& out, bool single_ok, Timer& tm, Issue issue,
                       PreLaunch pre_launch = PreLaunch()) {
    cudaStream_t st = g->stream;
    const bool stepwise = !g->opt_cuda_graph || g->opt_trace >= 2 || g->opt_timing || g->fab_host_bar;
    out.clear();
    // first iteration of a level: singleton fast path when rows hold distinct columns
    bool first_single = single_ok && g->opt_singleton;
    int log_base_host = 0;   // mirror of carry->log_base
    if (stepwise || first_single) {
        for (;;) {
            pre_launch();
            issue(0ull, first_single);
            CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
            const int slot = (int)out.size() - log_base_host;
            CK(cudaMemcpyAsync(wk.h_log, wk.log + slot, sizeof(IterLog), cudaMemcpyDeviceToHost, st));
            if (g->opt_trace >= 2) {
                g->trace_labels.emplace_back(g->cur_n);
                CK(cudaMemcpyAsync(g->trace_labels.back().data(), wk.C, sizeof(int32_t) * g->cur_n, cudaMemcpyDeviceToHost, st));
            }
            CK(cudaStreamSynchronize(st));
            tm.resolve();
            out.push_back(*wk.h_log);
            const Carry& c = *wk.h_carry;
            const bool cap_hit = g->opt_max_iters > 0 && c.iter >= g->opt_max_iters;
            if (c.converged || cap_hit) return;
            if (!c.more) {   // log full: restart slots at the current iteration
                log_base_host = c.iter;
                CK(cudaMemcpyAsync(&wk.carry->log_base, &log_base_host, sizeof(int), cudaMemcpyHostToDevice, st));
                CK(cudaStreamSynchronize(st));
            }
            first_single = false;
            if (!stepwise) break;   // continue in graph mode
        }
    }
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    CK(cudaGraphCreate(&graph, 0));
    try {
        cudaGraphConditionalHandle handle;
        CK(cudaGraphConditionalHandleCreate(&handle, graph, 1, cudaGraphCondAssignDefault));
        cudaGraphNodeParams cp = {};
        cp.type = cudaGraphNodeTypeConditional;
        cp.conditional.handle = handle;
        cp.conditional.type = cudaGraphCondTypeWhile;
        cp.conditional.size = 1;
        cudaGraphNode_t node;
        CK(cudaGraphAddNode(&node, graph, nullptr, 0, &cp));
        cudaGraph_t body = cp.conditional.phGraph_out[0];
        CK(cudaStreamBeginCaptureToGraph(st, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
        try {
            issue((unsigned long long)handle, false);
        } catch (...) {
            cudaGraph_t dummy;
            cudaStreamEndCapture(st, &dummy);
            throw;
        }
        CK(cudaStreamEndCapture(st, &body));
        CK(cudaGraphInstantiate(&exec, graph, 0));
        for (;;) {
            pre_launch();
            CK(cudaGraphLaunch(exec, st));
            CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            const Carry c = *wk.h_carry;
            const int first = (int)out.size() - log_base_host, last = c.iter - log_base_host;
            if (last > first)
                CK(cudaMemcpyAsync(wk.h_log, wk.log + first, sizeof(IterLog) * (last - first), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            for (int i = 0; i < last - first; ++i) out.push_back(wk.h_log[i]);
            const bool cap_hit = g->opt_max_iters > 0 && c.iter >= g->opt_max_iters;
            if (c.converged || cap_hit) break;
            log_base_host = c.iter;   // log full: continue with fresh slots
            CK(cudaMemcpyAsync(&wk.carry->log_base, &log_base_host, sizeof(int), cudaMemcpyHostToDevice, st));
        }
    } catch (...) {
        if (exec) cudaGraphExecDestroy(exec);
        cudaGraphDestroy(graph);
        throw;
    }
    cudaGraphExecDestroy(exec);
    cudaGraphDestroy(graph);
}

template <int M, bool UNIT>
static void phase1_level(gala_graph_s* g, Work& wk, const DevCSR& G, typename ModeT<M>::ST qW,
                         typename ModeT<M>::ST p, i128 qW128, i128 T, Timer& tm, int64_t maxdeg, int idbits,
                         std::vector<IterLog>& out, int level, bool single_ok) {
    block_setup<M, UNIT>(g);   // host-side attributes / grids before any capture (block_split may have changed)
    g->cur_n = G.n;
    (void)level;
    level_loop(g, wk, out, single_ok, tm, [&](unsigned long long cond, bool single) {
        issue_iteration<M, UNIT>(g, wk, G, qW, p, qW128, T, tm, maxdeg, idbits, cond, single);
    });
}

static i128 carry_N(const Carry* c) {
    return (i128)(((unsigned __int128)(ull)c->N_hi << 64) | (unsigned __int128)c->N_lo);
}
static i128 log_N(const IterLog& l) {
    return (i128)(((unsigned __int128)(ull)l.N_hi << 64) | (unsigned __int128)l.N_lo);
}

// algorithmic bytes per kernel class of one iteration
static void account_bytes(gala_graph_s* g, const IterCounters& c, int64_t n, int64_t nnz, bool unit, bool single) {
    const double om = unit ? 0.0 : 8.0;
    double act = 0;
    for (int b = 0; b < NBINS; ++b) {
        double cnt = (double)c.bin_count[b], deg = (double)c.bin_deg[b], kk = (double)c.bin_k[b];
        // per vertex: queue 4, row_ptr pair 16, C[v] 4, d 8, Sig[C[v]] 8, nextC 4; per entry: col 4 (+w), C[u] 4;
        // per distinct neighbour community: Sig 8
        int kc = b <= BIN_S32 ? KC_DEC_SMALL : KC_DEC_WARP + (b - BIN_WARP);
        if (single && kc != KC_DEC_HUB) kc = KC_DEC_SINGLE;   // first iteration: singleton kernels
        g->kc_bytes[kc] += cnt * (4 + 16 + 4 + 8 + 8 + 4) + deg * (4 + om + 4) + 8 * kk;
        act += cnt;
    }
    // prune: d, dp, C, Sig[C] per vertex; row_ptr pair + queue write per active
    g->kc_bytes[KC_PRUNE] += (double)n * (8 + 8 + 4 + 8) + act * (16 + 4);
    double m = (double)c.n_moved;
    // apply: queue + nextC + C per active; per mover C, stamp, d, 2 Sig, 2 size, row_ptr pair, list 8
    g->kc_bytes[KC_APPLY] += act * (4 + 4 + 4) + m * (4 + 4 + 8 + 16 + 8 + 16 + 8);
    if (c.delta_used)
        g->kc_bytes[KC_DP] += m * (8 + 16 + 4 + 8) + (double)c.moved_deg * (4 + om + 4 + 4);
    else
        g->kc_bytes[KC_DP] += (double)n * (16 + 4 + 8) + (double)nnz * (4 + om + 4);
    g->kc_bytes[KC_REDUCE] += (double)n * 24;
}

// verbose host-side phase timing (option "verbose"): synchronises the stream
struct VTimer {
    gala_graph_s* g;
    std::chrono::steady_clock::time_point t;
    explicit VTimer(gala_graph_s* gg) : g(gg), t(std::chrono::steady_clock::now()) {}
    void lap(const char* what) {
        if (!g->opt_verbose) return;
        cudaStreamSynchronize(g->stream);
        auto now = std::chrono::steady_clock::now();
        fprintf(stderr, "[gala] %-28s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(now - t).count());
        t = now;
    }
};

// ------------------------------------------------------------------ phase 2 (a9)
// Coarsen level graph `cur` with community ids newid[v] in [0, k) into `nxt`
// (reading c10: the diagonal carries D_C(c) once).  See k_phase2.cuh for
// the per-community aggregation paths.  Coarse d(c) = Sigma_tot(c), s(c) = diagonal.
#ifndef GALA_AGG_BT_C
#define GALA_AGG_BT_C 512    // threads of the largest block-path class (tables <= scap slots)
#endif
#ifndef GALA_AGG_BT_B
#define GALA_AGG_BT_B 256    // threads of the middle class (tables <= AGG_BB slots)
#endif
#define AGG_BLOCK_BT GALA_AGG_BT_C
template <typename V>
static size_t agg_block_smem(int scap) { return (size_t)scap * (sizeof(V) + sizeof(int)) + (size_t)(scap / 2) * sizeof(int); }

// warp / block aggregation launches with V = table value type (32-bit iff W < 2^32).
// The block path runs in three size classes so small tables get small blocks
// (more communities in flight per SM): <= AGG_BA slots with 128 threads,
// <= AGG_BB with 256, <= scap with 512.
template <int BT, bool UNIT, typename V>
static void agg_block_class(gala_graph_s* g, const AggArgs& a, int cap, const int32_t* bl, const int* nbl) {
    const size_t sm = agg_block_smem<V>(cap);
    CK(cudaFuncSetAttribute(k_agg_block<BT, UNIT, V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    int per = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_agg_block<BT, UNIT, V>, BT, sm));
    k_agg_block<BT, UNIT, V><<<g->num_sms * std::max(per, 1), BT, sm, g->stream>>>(a, cap, bl, nbl);
    CKL();
}

template <typename V>
static void agg_launch_small(gala_graph_s* g, const AggArgs& a, bool unit, int scap, long long k, const int32_t* wl,
                             const int* nwl, const int32_t* bl, const int* nbl) {
    cudaStream_t st = g->stream;
    const int big = g->num_sms * 8;
    if (unit) k_agg_warp<true, V><<<big, 256, 0, st>>>(a, wl, nwl);
    else k_agg_warp<false, V><<<big, 256, 0, st>>>(a, wl, nwl);
    CKL();
    const int ca = std::min(scap, AGG_BA), cb = std::min(scap, AGG_BB);
    if (scap > AGG_WSLOTS) {
        if (unit) agg_block_class<128, true, V>(g, a, ca, bl, nbl);
        else agg_block_class<128, false, V>(g, a, ca, bl, nbl);
    }
    if (scap > AGG_BA) {
        if (unit) agg_block_class<GALA_AGG_BT_B, true, V>(g, a, cb, bl + k, nbl + 1);
        else agg_block_class<GALA_AGG_BT_B, false, V>(g, a, cb, bl + k, nbl + 1);
    }
    if (scap > AGG_BB) {
        if (unit) agg_block_class<AGG_BLOCK_BT, true, V>(g, a, scap, bl + 2 * k, nbl + 2);
        else agg_block_class<AGG_BLOCK_BT, false, V>(g, a, scap, bl + 2 * k, nbl + 2);
    }
}

// Aggregate the rows of `cur` (nrows rows, each with a row-id array) into k
// target rows: target of row v is newid[v]; entries become (newid[u], w) and
// equal (target, key) pairs are summed.  Output CSR in pool memory with int64
// weights and row ids; snew[c] (caller-allocated, k) receives the diagonal.
// few communities: dense k x k accumulation (k_agg_dense_*); V = 32-bit iff W < 2^32
template <typename V>
static void aggregate_rows_dense(gala_graph_s* g, const DevCSR& cur, long long k, const int32_t* newid,
                                 const int32_t* keymap, bool unit, DevCSR& nxt, int64_t& maxdeg, int64_t* snew) {
    cudaStream_t st = g->stream;
    const int big = g->num_sms * 8;
    V* M = dalloc<V>((size_t)k * k, st);
    CK(cudaMemsetAsync(M, 0, sizeof(V) * (size_t)k * k, st));
    if (cur.nnz) {
        const int grid = grid_for((cur.nnz + 127) / 128 * 32, 256, big);
        if (unit) k_agg_dense_accum<true, V><<<grid, 256, 0, st>>>(cur.nnz, cur.row, cur.col, cur.w, newid, keymap, k, M);
        else k_agg_dense_accum<false, V><<<grid, 256, 0, st>>>(cur.nnz, cur.row, cur.col, cur.w, newid, keymap, k, M);
        CKL();
    }
    long long* dn = dalloc<long long>(k + 1, st);
    k_agg_dense_count<V><<<grid_for(k * 32, 256, big), 256, 0, st>>>(k, M, dn, snew);
    CKL();
    nxt.n = k;
    nxt.rp = dalloc<int64_t>(k + 1, st);
    scan_excl(dn, reinterpret_cast<long long*>(nxt.rp), k, st);
    ull* dev_max = dalloc<ull>(1, st);
    CK(cudaMemsetAsync(dev_max, 0, sizeof(ull), st));
    k_rowmax<<<grid_for(k, 256, big), 256, 0, st>>>(k, reinterpret_cast<long long*>(nxt.rp), dev_max);
    CKL();
    ull hm = 0;
    CK(cudaMemcpyAsync(&nxt.nnz, nxt.rp + k, sizeof(long long), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&hm, dev_max, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    maxdeg = (int64_t)hm;
    nxt.col = dalloc<int32_t>(nxt.nnz, st);
    nxt.w = dalloc<int64_t>(nxt.nnz, st);
    nxt.row = dalloc<int32_t>(nxt.nnz, st);
    k_agg_dense_emit<V><<<grid_for(k * 32, 256, big), 256, 0, st>>>(k, M, reinterpret_cast<long long*>(nxt.rp), nxt.col,
                                                                    nxt.w, nxt.row);
    CKL();
    g->kc_bytes[KC_PHASE2] += (double)cur.nnz * (4 + 4 + (unit ? 0 : 8) + 4) + (double)k * k * sizeof(V) * 2 +
                              (double)nxt.nnz * 16;
    dfree(M, st); dfree(dn, st); dfree(dev_max, st);
}

static void aggregate_rows(gala_graph_s* g, const DevCSR& cur, int64_t nrows, long long k, const int32_t* newid,
                           const int32_t* keymap, bool unit, DevCSR& nxt, int64_t& maxdeg, int64_t* snew) {
    cudaStream_t st = g->stream;
    const int big = g->num_sms * 8;
    VTimer vt(g);
    // few communities, many entries: dense accumulation (the coarse graph has at most k^2 entries)
    if (g->opt_agg_dense && k <= AGG_DENSE_K && (g->opt_agg_dense == 2 || cur.nnz >= 4 * k * k) && cur.row) {
        if (g->W < ((int64_t)1 << 32)) aggregate_rows_dense<unsigned>(g, cur, k, newid, keymap, unit, nxt, maxdeg, snew);
        else aggregate_rows_dense<ull>(g, cur, k, newid, keymap, unit, nxt, maxdeg, snew);
        vt.lap("agg: dense");
        return;
    }
    long long* cnt = dalloc<long long>(k + 1, st);
    long long* ent = dalloc<long long>(k + 1, st);
    long long* eoff = dalloc<long long>(k + 1, st);
    long long* dn = dalloc<long long>(k + 1, st);
    int* tkey = dalloc<int>(cur.nnz, st);
    // segment weights: 32-bit when W < 2^32 (every aggregated weight is <= W): halves the largest
    // phase-2 temporary (14.5 GB of 29 GB on the level-0 Friendster shape)
    TVal tval;
    tval.w32 = g->W < ((int64_t)1 << 32);
    tval.p = dalloc<char>((size_t)cur.nnz * (tval.w32 ? 4 : 8), st);
    ull* dev_max = dalloc<ull>(1, st);
    int32_t* bigc = dalloc<int32_t>(k, st);
    long long* bigcap = dalloc<long long>(k + 1, st);
    int32_t* wlist = dalloc<int32_t>(k, st);
    int32_t* blist = dalloc<int32_t>(4 * k, st);   // block-path classes A, B, C, D (spilling)
    int* nbig_dev = dalloc<int>(6, st);   // big, warp, block A / B / C / D list lengths
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (k + 1), st));
    CK(cudaMemsetAsync(ent, 0, sizeof(long long) * (k + 1), st));
    CK(cudaMemsetAsync(dn, 0, sizeof(long long) * (k + 1), st));
    CK(cudaMemsetAsync(snew, 0, sizeof(int64_t) * k, st));
    CK(cudaMemsetAsync(dev_max, 0, sizeof(ull), st));
    CK(cudaMemsetAsync(nbig_dev, 0, sizeof(int) * 6, st));
    const bool hist = k <= AGG_HIST_K;   // few communities: block-local histograms first
    const unsigned htiles = (unsigned)std::max<long long>((nrows + AGG_HIST_T - 1) / AGG_HIST_T, 1);
    if (hist) k_comm_stats_hist<<<htiles, 256, k * sizeof(unsigned), st>>>((int)nrows, k, cur.rp, newid, ent);
    else k_comm_stats<<<grid_for(nrows, 256, big), 256, 0, st>>>((int)nrows, cur.rp, newid, ent);
    CKL();
    scan_excl(ent, eoff, k, st);
    // segment position of every row (cnt reused as the per-community cursor), then an
    // edge-parallel copy of the keys keymap[u] into the segments
    long long* vpos = dalloc<long long>(nrows, st);
    if (hist)
        k_vpos_hist<<<htiles, 256, ((k * sizeof(unsigned) + 15) & ~(size_t)15) + k * sizeof(long long), st>>>(
            (int)nrows, k, cur.rp, newid, eoff, cnt, vpos);
    else k_vpos<<<grid_for(nrows, 256, big), 256, 0, st>>>((int)nrows, cur.rp, newid, eoff, cnt, vpos);
    CKL();
    if (unit)
        k_gather_flat<true><<<grid_for((cur.nnz + 127) / 128 * 32, 256, big), 256, 0, st>>>(
            cur.nnz, cur.row, cur.rp, cur.col, cur.w, keymap, vpos, tkey, tval);
    else
        k_gather_flat<false><<<grid_for((cur.nnz + 127) / 128 * 32, 256, big), 256, 0, st>>>(
            cur.nnz, cur.row, cur.rp, cur.col, cur.w, keymap, vpos, tkey, tval);
    CKL();
    dfree(vpos, st);
    vt.lap("agg: stats+gather");
    // shared-memory capacity of the block path: up to 8192 slots (14 B each)
    int scap = 512;
    while (scap < g->opt_agg_scap && scap < 2 * k) scap <<= 1;
    const long long spill_ent = g->opt_agg_spill ? g->opt_agg_big_ent : 0;
    k_agg_classify<<<grid_for(k, 256, big), 256, 0, st>>>(k, ent, scap, dn, wlist, nbig_dev + 1, blist, nbig_dev + 2,
                                                         bigc, bigcap, nbig_dev, k, g->opt_agg_big_ent, spill_ent);
    CKL();
    AggArgs a;
    a.k = k; a.ent = ent; a.eoff = eoff; a.tkey = tkey; a.tval = tval; a.dn = dn; a.snew = snew;
    const bool v32 = g->W < ((int64_t)1 << 32);   // every aggregated weight is <= W
    if (v32) agg_launch_small<unsigned>(g, a, unit, scap, k, wlist, nbig_dev + 1, blist, nbig_dev + 2);
    else agg_launch_small<ull>(g, a, unit, scap, k, wlist, nbig_dev + 1, blist, nbig_dev + 2);
    vt.lap("agg: warp+block");
    int hcnt[6] = {0, 0, 0, 0, 0, 0};
    CK(cudaMemcpyAsync(hcnt, nbig_dev, sizeof(hcnt), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const int nbig = hcnt[0];
    if (hcnt[5] > 0) {   // class D: shared H0 spilling to per-block global H1 tables
        long long gcap = 64;
        while (gcap < 2 * std::min<long long>(spill_ent, k)) gcap <<= 1;
        const size_t sm = (size_t)scap * (v32 ? sizeof(unsigned) : sizeof(ull)) + (size_t)scap * 2 * sizeof(int);
        auto kf = unit ? (v32 ? (void*)k_agg_block_h<true, unsigned> : (void*)k_agg_block_h<true, ull>)
                       : (v32 ? (void*)k_agg_block_h<false, unsigned> : (void*)k_agg_block_h<false, ull>);
        CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
        int per = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kf, 512, sm));
        const int gd = (int)std::min<long long>((long long)g->num_sms * std::max(per, 1), hcnt[5]);
        int* hk = dalloc<int>((size_t)gd * gcap, st);
        ull* hv = dalloc<ull>((size_t)gd * gcap, st);
        int* hl = dalloc<int>((size_t)gd * gcap, st);
        CK(cudaMemsetAsync(hk, 0xff, sizeof(int) * (size_t)gd * gcap, st));
        CK(cudaMemsetAsync(hv, 0, sizeof(ull) * (size_t)gd * gcap, st));
        const int32_t* bld = blist + 3 * k;
        if (unit && v32) k_agg_block_h<true, unsigned><<<gd, 512, sm, st>>>(a, scap, bld, nbig_dev + 5, hk, hv, hl, gcap);
        else if (unit) k_agg_block_h<true, ull><<<gd, 512, sm, st>>>(a, scap, bld, nbig_dev + 5, hk, hv, hl, gcap);
        else if (v32) k_agg_block_h<false, unsigned><<<gd, 512, sm, st>>>(a, scap, bld, nbig_dev + 5, hk, hv, hl, gcap);
        else k_agg_block_h<false, ull><<<gd, 512, sm, st>>>(a, scap, bld, nbig_dev + 5, hk, hv, hl, gcap);
        CKL();
        dfree(hk, st); dfree(hv, st); dfree(hl, st);
        vt.lap("agg: spilling block");
    }
    if (nbig > 0 && g->opt_agg_big_chunk && g->opt_agg_bound) {
        // two-pass: chunk combine in place -> tables sized from the chunks' distinct counts
        const int ch = g->opt_agg_chunk;
        long long* nch = dalloc<long long>(nbig + 1, st);
        long long* choff = dalloc<long long>(nbig + 1, st);
        k_agg_big_nchunks<<<grid_for(nbig, 256, big), 256, 0, st>>>(nbig, bigc, ent, nch, ch);
        CKL();
        scan_excl(nch, choff, nbig, st);
        int* ndc = dalloc<int>(cur.nnz / ch + nbig + 1, st);   // >= total chunks
        const int gb = g->num_sms * 2;
        if (unit || v32) {
            const size_t sm = agg_chunk_smem<unsigned>();
            auto kf = unit ? k_agg_big_combine<true, unsigned> : k_agg_big_combine<false, unsigned>;
            CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
            kf<<<gb, 256, sm, st>>>(a, bigc, nbig, choff, ndc, ch);
        } else {
            const size_t sm = agg_chunk_smem<ull>();
            CK(cudaFuncSetAttribute(k_agg_big_combine<false, ull>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
            k_agg_big_combine<false, ull><<<gb, 256, sm, st>>>(a, bigc, nbig, choff, ndc, ch);
        }
        CKL();
        k_agg_big_bound<<<grid_for((long long)nbig * 32, 256, big), 256, 0, st>>>(nbig, k, choff, ndc, bigcap);
        CKL();
        vt.lap("agg: big combine");
        long long* goff = dalloc<long long>(nbig + 1, st);
        scan_excl(bigcap, goff, nbig, st);
        long long gtot = 0;
        CK(cudaMemcpyAsync(&gtot, goff + nbig, sizeof(long long), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        int* gkeys = dalloc<int>(gtot, st);
        // table values 32-bit whenever W < 2^32 (every aggregated weight is <= W)
        const size_t gvb = v32 ? sizeof(unsigned) : sizeof(ull);
        char* gvals = dalloc<char>((size_t)gtot * gvb, st);
        int* glist = dalloc<int>(gtot / 2 + 1, st);
        int* gcnt = dalloc<int>(nbig, st);
        CK(cudaMemsetAsync(gkeys, 0xff, sizeof(int) * gtot, st));
        CK(cudaMemsetAsync(gvals, 0, gvb * gtot, st));
        CK(cudaMemsetAsync(gcnt, 0, sizeof(int) * nbig, st));
        vt.lap("agg: big alloc+clear");
        if (v32) {
            k_agg_big_insert2<unsigned><<<big, 256, 0, st>>>(a, bigc, nbig, choff, ndc, ch, goff, gkeys,
                                                             reinterpret_cast<unsigned*>(gvals), glist, gcnt);
            CKL();
            vt.lap("agg: big insert");
            k_agg_big_emit2<unsigned><<<big, 256, 0, st>>>(a, bigc, nbig, choff, goff, gkeys,
                                                           reinterpret_cast<unsigned*>(gvals), glist, gcnt, ch);
        } else {
            k_agg_big_insert2<ull><<<big, 256, 0, st>>>(a, bigc, nbig, choff, ndc, ch, goff, gkeys,
                                                        reinterpret_cast<ull*>(gvals), glist, gcnt);
            CKL();
            vt.lap("agg: big insert");
            k_agg_big_emit2<ull><<<big, 256, 0, st>>>(a, bigc, nbig, choff, goff, gkeys, reinterpret_cast<ull*>(gvals),
                                                      glist, gcnt, ch);
        }
        CKL();
        dfree(nch, st); dfree(choff, st); dfree(ndc, st);
        dfree(goff, st); dfree(gkeys, st); dfree(gvals, st); dfree(glist, st); dfree(gcnt, st);
        if (g->opt_verbose) fprintf(stderr, "[gala] big communities %d, table slots %lld (bounded)\n", nbig, gtot);
    } else if (nbig > 0) {
        long long* goff = dalloc<long long>(nbig + 1, st);
        scan_excl(bigcap, goff, nbig, st);
        long long gtot = 0;
        CK(cudaMemcpyAsync(&gtot, goff + nbig, sizeof(long long), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        int* gkeys = dalloc<int>(gtot, st);
        ull* gvals = dalloc<ull>(gtot, st);
        int* glist = dalloc<int>(gtot / 2 + 1, st);
        int* gcnt = dalloc<int>(nbig, st);
        CK(cudaMemsetAsync(gkeys, 0xff, sizeof(int) * gtot, st));
        CK(cudaMemsetAsync(gvals, 0, sizeof(ull) * gtot, st));
        CK(cudaMemsetAsync(gcnt, 0, sizeof(int) * nbig, st));
        vt.lap("agg: big alloc+clear");
        long long* nch = dalloc<long long>(nbig + 1, st);
        long long* choff = dalloc<long long>(nbig + 1, st);
        k_agg_big_nchunks<<<grid_for(nbig, 256, big), 256, 0, st>>>(nbig, bigc, ent, nch, g->opt_agg_chunk);
        CKL();
        scan_excl(nch, choff, nbig, st);
        if (g->opt_agg_big_chunk) {
            const int gb = g->num_sms * 2;   // 80 KB (32-bit values) / 112 KB smem per block
            if (unit || v32) {
                const size_t sm = agg_chunk_smem<unsigned>();
                auto kf = unit ? k_agg_big_chunk<true, unsigned> : k_agg_big_chunk<false, unsigned>;
                CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
                kf<<<gb, 256, sm, st>>>(a, bigc, nbig, choff, goff, gkeys, gvals, glist, gcnt, g->opt_agg_chunk);
            } else {
                const size_t sm = agg_chunk_smem<ull>();
                CK(cudaFuncSetAttribute(k_agg_big_chunk<false, ull>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
                k_agg_big_chunk<false, ull><<<gb, 256, sm, st>>>(a, bigc, nbig, choff, goff, gkeys, gvals, glist, gcnt,
                                                                g->opt_agg_chunk);
            }
            CKL();
            vt.lap("agg: big insert");
            k_agg_big_emit2<ull><<<big, 256, 0, st>>>(a, bigc, nbig, choff, goff, gkeys, gvals, glist, gcnt, g->opt_agg_chunk);
            CKL();
        } else {
            const int bpc = 32;
            if (unit) k_agg_big_insert<true, unsigned><<<big, 256, 0, st>>>(a, bigc, nbig, goff, gkeys, gvals, glist, gcnt, bpc);
            else if (v32) k_agg_big_insert<false, unsigned><<<big, 256, 0, st>>>(a, bigc, nbig, goff, gkeys, gvals, glist, gcnt, bpc);
            else k_agg_big_insert<false, ull><<<big, 256, 0, st>>>(a, bigc, nbig, goff, gkeys, gvals, glist, gcnt, bpc);
            CKL();
            vt.lap("agg: big insert");
            k_agg_big_emit<<<big, 256, 0, st>>>(a, bigc, nbig, goff, gkeys, gvals, glist, gcnt, bpc);
            CKL();
        }
        dfree(nch, st); dfree(choff, st);
        dfree(goff, st); dfree(gkeys, st); dfree(gvals, st); dfree(glist, st); dfree(gcnt, st);
        if (g->opt_verbose) fprintf(stderr, "[gala] big communities %d, table slots %lld\n", nbig, gtot);
    }
    vt.lap("agg: big");
    nxt.n = k;
    nxt.rp = dalloc<int64_t>(k + 1, st);
    scan_excl(dn, reinterpret_cast<long long*>(nxt.rp), k, st);
    k_rowmax<<<grid_for(k, 256, big), 256, 0, st>>>(k, reinterpret_cast<long long*>(nxt.rp), dev_max);
    CKL();
    ull hm = 0;
    CK(cudaMemcpyAsync(&nxt.nnz, nxt.rp + k, sizeof(long long), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&hm, dev_max, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    maxdeg = (int64_t)hm;
    nxt.col = dalloc<int32_t>(nxt.nnz, st);
    nxt.w = dalloc<int64_t>(nxt.nnz, st);
    nxt.row = dalloc<int32_t>(nxt.nnz, st);
    vt.lap("agg: scan+alloc");
    if (nxt.nnz > 0) {
        int32_t* tmap = dalloc<int32_t>((nxt.nnz + 255) / 256, st);
        k_tile_map<<<grid_for(k, 256, big), 256, 0, st>>>(k, reinterpret_cast<long long*>(nxt.rp), nxt.nnz, tmap);
        CKL();
        k_compact<<<grid_for((nxt.nnz + 255) / 256, 1, big * 2), 256, 0, st>>>(
            k, nxt.nnz, eoff, reinterpret_cast<long long*>(nxt.rp), tmap, tkey, tval, nxt.col, nxt.w, nxt.row);
        CKL();
        dfree(tmap, st);
    }
    vt.lap("agg: scan+compact");
    g->kc_bytes[KC_PHASE2] += (double)nrows * (4 + 4 + 8 + 16 + 4 + 4) + (double)cur.nnz * (4 + 4 + (unit ? 0 : 8) + 12) +
                              (double)nxt.nnz * 24;
    dfree(cnt, st); dfree(ent, st); dfree(eoff, st); dfree(dn, st);
    { char* tp = static_cast<char*>(tval.p); dfree(tp, st); }
    dfree(tkey, st); dfree(dev_max, st); dfree(bigc, st);
    dfree(bigcap, st); dfree(nbig_dev, st); dfree(wlist, st); dfree(blist, st);
}

// ------------------------------------------------------------------ phase 2 (a9)
// Coarsen level graph `cur` with community ids newid[v] in [0, k) into `nxt`
// (reading c10: the diagonal carries D_C(c) once).  Coarse d(c) =
// Sigma_tot(c) (maintained exactly by phase 1), s(c) = the diagonal.
static void coarsen(gala_graph_s* g, Work& wk, const DevCSR& cur, int64_t nl, long long k, const int32_t* newid,
                    const int32_t* minmem, bool unit, DevCSR& nxt, int64_t& maxdeg, int64_t& dmax) {
    cudaStream_t st = g->stream;
    const int big = g->num_sms * 8;
    int64_t* snew = dalloc<int64_t>(k, st);
    int64_t* dnew = dalloc<int64_t>(k, st);
    ull* dev_max = dalloc<ull>(1, st);
    aggregate_rows(g, cur, nl, k, newid, newid, unit, nxt, maxdeg, snew);
    CK(cudaMemsetAsync(dev_max, 0, sizeof(ull), st));
    k_coarsen_deg<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, newid, wk.Sig, dnew);
    CKL();
    k_max_i64<<<grid_for(k, 256, big), 256, 0, st>>>(k, dnew, dev_max);
    CKL();
    ull hm = 0;
    CK(cudaMemcpyAsync(&hm, dev_max, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(wk.d, dnew, sizeof(int64_t) * k, cudaMemcpyDeviceToDevice, st));
    CK(cudaMemcpyAsync(wk.s, snew, sizeof(int64_t) * k, cudaMemcpyDeviceToDevice, st));
    wk.s_zero = false;
    CK(cudaStreamSynchronize(st));
    dmax = (int64_t)hm;
    dfree(snew, st);
    dfree(dnew, st);
    dfree(dev_max, st);
}

// Final numerator.  The last level's N equals N of the composed labels on the
// level-0 graph (coarsening preserves Q exactly, invariant P4); with option
// "check" it is recomputed on G0 from the labels (Eq. 1) and compared.
static void final_numerator(gala_graph_s* g, int64_t p, int64_t q, int64_t W, i128 N_last) {
    g->N = N_last;
    g->check_mismatch = 0;
    if (!g->opt_check) return;
    cudaStream_t st = g->stream;
    const int64_t n0 = g->n0;
    const int big = g->num_sms * 8;
    long long* DV = dalloc<long long>(n0, st);
    ull* DC = dalloc<ull>(1, st);
    i128* part = dalloc<i128>(big, st);
    ull* ticket = dalloc<ull>(1, st);
    i128* out = dalloc<i128>(1, st);
    CK(cudaMemsetAsync(DV, 0, sizeof(long long) * n0, st));
    CK(cudaMemsetAsync(DC, 0, sizeof(ull), st));
    CK(cudaMemsetAsync(ticket, 0, sizeof(ull), st));
    if (g->g0.w == nullptr)
        k_mod_dc<true><<<big, 256, 0, st>>>((int)n0, g->g0.rp, g->g0.col, g->g0.w, g->lab, g->d0, DV, DC);
    else
        k_mod_dc<false><<<big, 256, 0, st>>>((int)n0, g->g0.rp, g->g0.col, g->g0.w, g->lab, g->d0, DV, DC);
    CKL();
    k_sumsq<<<grid_for(n0, 256, big), 256, 0, st>>>(n0, DV, part, ticket, out);
    CKL();
    ull hdc = 0;
    i128 hs2 = 0;
    CK(cudaMemcpyAsync(&hdc, DC, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&hs2, out, sizeof(i128), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const i128 N0 = (i128)q * W * (i128)(long long)hdc - (i128)p * hs2;
    if (N0 != N_last) g->check_mismatch = 1;
    dfree(DV, st); dfree(DC, st); dfree(part, st); dfree(ticket, st); dfree(out, st);
}

// ------------------------------------------------------------------ the multi-level run
// The run workspace (sized for level 0) is allocated once per handle and reused by every run.
static void ensure_workspace(gala_graph_s* g) {
    cudaStream_t st = g->stream;
    const int64_t n0 = g->n0;
    if (g->wk && g->wk->log_cap != g->opt_log_cap) { g->wk->release(); delete g->wk; g->wk = nullptr; }
    if (!g->wk) {
        g->wk = new Work();
        Work& wk = *g->wk;
        wk.st = st;
        wk.ncap = std::max<int64_t>(n0, 1);
        wk.nnzcap = g->nnz0;
        wk.log_cap = g->opt_log_cap;
        try {
            wk.C = dalloc<int32_t>(wk.ncap, st);
            wk.size = dalloc<int32_t>(wk.ncap, st);
            wk.stamp = dalloc<int32_t>(wk.ncap, st);
            wk.cst = dalloc<int2>(wk.ncap, st);
            // delta-update items: one per light mover + one per DCH-entry chunk of a heavy one
            const size_t icap = (size_t)wk.ncap + (size_t)(g->nnz0 / DCH) + 1;
            wk.icap = (long long)icap;
            wk.mv_v = dalloc<int32_t>(icap, st);
            wk.mv_old = dalloc<int32_t>(icap, st);
            wk.mv_chunk = dalloc<int32_t>(icap, st);
            wk.nextC = dalloc<int32_t>(wk.ncap, st);
            // multi-GPU: only owned vertices are queued (largest owned range; grown per level if needed)
            wk.qcap = wk.ncap;
            if (g->di && g->dbounds0.size() > 1) {
                long long mx = 1;
                for (size_t r = 0; r + 1 < g->dbounds0.size(); ++r) mx = std::max(mx, g->dbounds0[r + 1] - g->dbounds0[r]);
                wk.qcap = mx;
            }
            wk.queues = dalloc<QRec>((size_t)wk.qcap * (NBINS / 2), st);
            if (g->ckey_ok) wk.ckey = dalloc<int32_t>(g->nnz0, st);
            wk.Sig = dalloc<int64_t>(wk.ncap, st);
            wk.d = dalloc<int64_t>(wk.ncap, st);
            wk.s = dalloc<int64_t>(wk.ncap, st);
            wk.dp = dalloc<int64_t>(wk.ncap, st);
            wk.ctr = dalloc<IterCounters>(1, st);
            wk.carry = dalloc<Carry>(1, st);
            wk.log = dalloc<IterLog>(wk.log_cap, st);
            wk.reduce_grid = g->num_sms * 4;
            wk.part_dc = dalloc<long long>(wk.reduce_grid, st);
            wk.part_min = dalloc<long long>(wk.reduce_grid, st);
            wk.part_s2 = dalloc<i128>(wk.reduce_grid, st);
            wk.h_log = static_cast<IterLog*>(pin_get(sizeof(IterLog) * (size_t)wk.log_cap));
            wk.h_carry = static_cast<Carry*>(pin_get(sizeof(Carry)));
            if (!wk.h_log || !wk.h_carry) { set_err(GALA_E_NOMEM, "pinned host buffers"); throw GalaError{GALA_E_NOMEM}; }
            for (int i = 0; i < 5; ++i) CK(cudaEventCreate(&wk.ev[i]));
            // dynamic shared memory opt-ins (process-wide upper bounds, set once)
            int per_sm = 0;
            const int cap = g->hub_smem_slots;
            block_attrs_ensure(block_arena_slots(g));
            // resident blocks per SM of each mode's block kernel (the grid of a launch; spill
            // tables are sized for the largest)
            auto occ = [&](const void* f, size_t sm) {
                int b = 0;
                CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, f, BLOCK_BT, sm));
                return std::max(b, 1);
            };
            wk.gblocks_m[DM_FAST] = g->num_sms * std::min(occ((const void*)k_decide_block<BLOCK_BT, BLOCK_E, DM_FAST, true>, block_smem_bytes<DM_FAST>(cap)),
                                                          occ((const void*)k_decide_block<BLOCK_BT, BLOCK_E, DM_FAST, false>, block_smem_bytes<DM_FAST>(cap)));
            wk.gblocks_m[DM_W64] = g->num_sms * std::min(occ((const void*)k_decide_block<BLOCK_BT, BLOCK_E, DM_W64, true>, block_smem_bytes<DM_W64>(cap)),
                                                         occ((const void*)k_decide_block<BLOCK_BT, BLOCK_E, DM_W64, false>, block_smem_bytes<DM_W64>(cap)));
            wk.gblocks_m[DM_W128] = g->num_sms * std::min(occ((const void*)k_decide_block<BLOCK_BT, BLOCK_E, DM_W128, true>, block_smem_bytes<DM_W128>(cap)),
                                                          occ((const void*)k_decide_block<BLOCK_BT, BLOCK_E, DM_W128, false>, block_smem_bytes<DM_W128>(cap)));
            per_sm = std::max(std::max(wk.gblocks_m[0], wk.gblocks_m[1]), wk.gblocks_m[2]) / g->num_sms;
            set_warp_smem<32, 128, DM_FAST>(); set_warp_smem<32, 128, DM_W64>(); set_warp_smem<32, 128, DM_W128>();
            set_warp_smem<32, 512, DM_FAST>(); set_warp_smem<32, 512, DM_W64>(); set_warp_smem<32, 512, DM_W128>();
            wk.gblocks = g->num_sms * std::max(per_sm, 1);
            wk.gcap = 0;   // spill tables sized on demand (coarse levels can have larger rows than level 0)
            wk.smem_cap = cap;
        } catch (...) {
            wk.release();
            delete g->wk;
            g->wk = nullptr;
            throw;
        }
    }
}


static void do_run(gala_graph_s* g, double gamma, double tol, int max_levels) {
    PoolScope pool_scope(g->cache);
    cudaStream_t st = g->stream;
    CK(cudaSetDevice(g->device));
    g->has_result = false;
    g->trace.clear();
    g->trace_labels.clear();
    g->levels.clear();
    for (int i = 0; i < KC_COUNT; ++i) { g->kc_ms[i] = 0; g->kc_bytes[i] = 0; g->kc_launches[i] = 0; }
    for (double& x : g->tbl) x = 0;
    g->dp_mismatch = 0;
    const long long launches0 = g_launches;
    int64_t p, q;
    gamma_to_pq(gamma, &p, &q);
    g->p = p;
    g->q = q;
    const int64_t n0 = g->n0, W = g->W;
    const int64_t mpq = std::max(p, q);
    if ((long double)mpq * (long double)W * (long double)W >= 0x1p125L) {
        set_err(GALA_E_OVERFLOW, "max(p,q)*W^2 >= 2^125");
        throw GalaError{GALA_E_OVERFLOW};
    }
    const i128 qW128 = (i128)q * W;
    const i128 T = (i128)ceill((long double)tol * (long double)q * (long double)W * (long double)W);

    const int big = g->num_sms * 8;
    if (!g->lab) g->lab = dalloc<int32_t>(n0, st);
    ensure_workspace(g);
    Work& wk = *g->wk;
    // option l2_window: keep the label array C (the per-entry random gathers) persisting in L2
    // through a stream access-policy window (matters once C + Sigma_tot outgrow the 126 MB L2)
    struct L2Window {
        cudaStream_t st = nullptr;
        ~L2Window() {
            if (!st) return;
            cudaStreamAttrValue v = {};
            v.accessPolicyWindow.num_bytes = 0;
            cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v);
            cudaCtxResetPersistingL2Cache();
        }
    } l2w;
    if (g->opt_l2_window) {
        int maxwin = 0, maxpers = 0;
        CK(cudaDeviceGetAttribute(&maxwin, cudaDevAttrMaxAccessPolicyWindowSize, g->device));
        CK(cudaDeviceGetAttribute(&maxpers, cudaDevAttrMaxPersistingL2CacheSize, g->device));
        const size_t bytes = std::min<size_t>((size_t)n0 * sizeof(int32_t), (size_t)std::max(maxwin, 0));
        CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min<size_t>(bytes, (size_t)std::max(maxpers, 0))));
        cudaStreamAttrValue v = {};
        v.accessPolicyWindow.base_ptr = wk.C;
        v.accessPolicyWindow.num_bytes = bytes;
        v.accessPolicyWindow.hitRatio = 1.0f;
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        CK(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v));
        l2w.st = st;
    }
    cudaEvent_t ev_run0 = wk.ev[0], ev_run1 = wk.ev[1];
    CK(cudaEventRecord(ev_run0, st));
    try {
        CK(cudaMemsetAsync(wk.ctr, 0, sizeof(IterCounters), st));
        CK(cudaMemsetAsync(wk.carry, 0, sizeof(Carry), st));
        DevCSR cur = g->g0;
        bool cur_owned = false;
        CK(cudaMemcpyAsync(wk.d, g->d0, sizeof(int64_t) * n0, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(wk.s, g->s0, sizeof(int64_t) * n0, cudaMemcpyDeviceToDevice, st));
        wk.s_zero = !g->self0;
        int64_t maxdeg = g->maxdeg0, dmax = g->maxw0;
        bool first_level = true;
        Timer tm(g);
        std::vector<IterLog> logs;
        for (int level = 0;; ++level) {
            const int64_t nl = cur.n;
            const bool unit = (cur.w == nullptr);
            LevelStat ls{};
            ls.n = nl;
            ls.nnz = cur.nnz;
            ls.maxdeg = maxdeg;
            cudaEvent_t lv0 = wk.ev[2], lv1 = wk.ev[3], lv2 = wk.ev[4];
            CK(cudaEventRecord(lv0, st));
            prepare_level_tables(g, wk, cur, maxdeg);
            // a1: level init + starting numerator
            cudaEvent_t e = tm.begin();
            k_level_init<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.d, wk.C, wk.Sig, wk.size, wk.dp, wk.stamp, wk.cst,
                                                                 wk.carry, prune_state(g, wk));
            CKL();
            if (first_level) {
                // lab = identity on level 0 (C is the identity right now)
                CK(cudaMemcpyAsync(g->lab, wk.C, sizeof(int32_t) * n0, cudaMemcpyDeviceToDevice, st));
                if (use_ckey(g, wk, cur) && cur.nnz) {
                    k_ckey_init<<<grid_for(cur.nnz, 256, big), 256, 0, st>>>(cur.nnz, cur.row, cur.col, wk.ckey,
                                                                             wk.carry);
                    CKL();
                }
                first_level = false;
            }
            k_iter_begin<<<1, 128, 0, st>>>(wk.ctr);
            CKL();
            k_reduce<256><<<wk.reduce_grid, 256, 0, st>>>((int)nl, 0, (int)nl, wk.dp, wk.s_live(), wk.Sig, wk.part_dc, wk.part_s2,
                                                          wk.part_min, wk.ctr, wk.carry, (long long)(qW128 >> 64),
                                                          (ull)qW128, (long long)p, 0, 0, 0);
            CKL();
            tm.end(KC_INIT, e);
            CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            const i128 N_start = carry_N(wk.h_carry);
            const ull t_level = wk.h_carry->t_ns;
            // gain arithmetic for this level (reading c16):
            //   |score| <= max(p,q) * W * dmax  (dmax = max weighted degree of the level)
            //   int64 iff that bound < 2^62; packed (score,-c) keys iff < 2^(62 - idbits); the
            //   int64 modes sum per-vertex aggregates in 32 bits, so they also need dmax < 2^32
            //   (else the int128 mode, whose aggregates are 64-bit).
            int idbits = 1;
            while (idbits < 31 && ((int64_t)1 << idbits) < nl) ++idbits;
            const long double bound = (long double)mpq * (long double)W * (long double)std::max<int64_t>(dmax, 1);
            int mode = DM_FAST;
            if (g->opt_force_i128 || bound >= 0x1p62L || dmax >= ((int64_t)1 << 32)) mode = DM_W128;
            else if (bound * (long double)((int64_t)1 << idbits) >= 0x1p62L || g->opt_force_wide)
                mode = DM_W64;
            ls.i128path = mode;
            const long long qW64 = (long long)qW128, p64 = (long long)p;
            if (mode == DM_W128) {
                if (unit) phase1_level<DM_W128, true>(g, wk, cur, (i128)qW128, (i128)p, qW128, T, tm, maxdeg, idbits, logs, level, level > 0 || g->rows_distinct0);
                else phase1_level<DM_W128, false>(g, wk, cur, (i128)qW128, (i128)p, qW128, T, tm, maxdeg, idbits, logs, level, level > 0 || g->rows_distinct0);
            } else if (mode == DM_W64) {
                if (unit) phase1_level<DM_W64, true>(g, wk, cur, qW64, p64, qW128, T, tm, maxdeg, idbits, logs, level, level > 0 || g->rows_distinct0);
                else phase1_level<DM_W64, false>(g, wk, cur, qW64, p64, qW128, T, tm, maxdeg, idbits, logs, level, level > 0 || g->rows_distinct0);
            } else {
                if (unit) phase1_level<DM_FAST, true>(g, wk, cur, qW64, p64, qW128, T, tm, maxdeg, idbits, logs, level, level > 0 || g->rows_distinct0);
                else phase1_level<DM_FAST, false>(g, wk, cur, qW64, p64, qW128, T, tm, maxdeg, idbits, logs, level, level > 0 || g->rows_distinct0);
            }
            i128 N = N_start;
            ull t_prev = t_level;
            for (size_t it = 0; it < logs.size(); ++it) {
                const IterCounters& c = logs[it].ctr;
                double b0 = 0, b1 = 0;
                for (int i = 0; i < KC_COUNT; ++i) b0 += g->kc_bytes[i];
                account_bytes(g, c, nl, cur.nnz, unit, it == 0 && g->opt_singleton && (level > 0 || g->rows_distinct0));
                g->tbl[0] += (double)c.h0_acc; g->tbl[1] += (double)c.h1_acc;
                g->tbl[2] += (double)c.h0_keys; g->tbl[3] += (double)c.h1_keys;
                for (int i = 0; i < KC_COUNT; ++i) b1 += g->kc_bytes[i];
                ls.alg_bytes += b1 - b0;
                const int64_t it_ns = logs[it].t_ns >= t_prev ? (int64_t)(logs[it].t_ns - t_prev) : 0;
                t_prev = logs[it].t_ns;
                g->dp_mismatch += (int64_t)c.dp_mismatch;
                N = log_N(logs[it]);
                int64_t scanned = 0, kk = 0;
                for (int b = 0; b < NBINS; ++b) { scanned += (int64_t)c.bin_deg[b]; kk += (int64_t)c.bin_k[b]; }
                ls.edges_scanned += scanned;
                ls.nominal_edges += cur.nnz;
                if (g->opt_trace >= 1) {
                    TraceRec r;
                    r.v[0] = level; r.v[1] = (int64_t)it; r.v[2] = nl; r.v[3] = (int64_t)c.n_active;
                    r.v[4] = (int64_t)c.n_pruned; r.v[5] = (int64_t)c.n_moved;
                    r.v[6] = (int64_t)(N >> 64); r.v[7] = (int64_t)(uint64_t)N;
                    r.v[8] = scanned; r.v[9] = kk; r.v[10] = (int64_t)c.delta_used; r.v[11] = 0;
                    r.v[12] = (int64_t)c.n_fn; r.v[13] = (int64_t)c.n_fp; r.v[14] = it_ns; r.v[15] = (int64_t)(b1 - b0);
                    g->trace.push_back(r);
                }
            }
            ls.iters = (int64_t)logs.size();
            ls.ms_iters = logs.empty() ? 0.0 : (double)(logs.back().t_ns - t_level) * 1e-6;
            CK(cudaEventRecord(lv1, st));
            // a8: relabel in min-member order + compose
            e = tm.begin();
            int32_t* minmem = dalloc<int32_t>(nl, st);
            long long* pos = dalloc<long long>(nl + 1, st);
            int32_t* newid = dalloc<int32_t>(nl, st);
            k_fill_i32<<<grid_for(nl, 256, big), 256, 0, st>>>(minmem, nl, INT_MAX);
            CKL();
            k_minmember<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem);
            CKL();
            k_minflag<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, pos);
            CKL();
            scan_excl(pos, pos, nl, st);
            k_newid<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, pos, newid);
            CKL();
            k_compose<<<grid_for(n0, 256, big), 256, 0, st>>>(n0, newid, g->lab);
            CKL();
            long long kcomm = 0;
            CK(cudaMemcpyAsync(&kcomm, pos + nl, sizeof(long long), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            g->k_final = kcomm;   // canonical final labels are 0..k-1 (reading c19)
            const bool stop = (kcomm == nl) || (max_levels > 0 && level + 1 >= max_levels) || (N - N_start < T);
            DevCSR nxt;
            if (!stop) coarsen(g, wk, cur, nl, kcomm, newid, minmem, unit, nxt, maxdeg, dmax);
            dfree(minmem, st);
            dfree(pos, st);
            dfree(newid, st);
            tm.end(KC_PHASE2, e);
            CK(cudaEventRecord(lv2, st));
            CK(cudaEventSynchronize(lv2));
            tm.resolve();
            float ms1 = 0, ms2 = 0;
            CK(cudaEventElapsedTime(&ms1, lv0, lv1));
            CK(cudaEventElapsedTime(&ms2, lv1, lv2));
            ls.ms_phase1 = ms1;
            ls.ms_phase2 = ms2;
            g->levels.push_back(ls);
            if (cur_owned) { dfree(cur.rp, st); dfree(cur.col, st); dfree(cur.w, st); dfree(cur.row, st); }
            if (stop) break;
            cur = nxt;
            cur_owned = true;
        }
        {
            i128 N_last = 0;
            CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            N_last = carry_N(wk.h_carry);
            final_numerator(g, p, q, W, N_last);
        }
        CK(cudaEventRecord(ev_run1, st));
        CK(cudaEventSynchronize(ev_run1));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, ev_run0, ev_run1));
        g->run_ms = ms;
        g->launches = g_launches - launches0;
        if (g->opt_verbose && g->cache) {
            unsigned long long res = 0, used = 0;
            cudaMemPoolGetAttribute(g->cache->pool, cudaMemPoolAttrReservedMemCurrent, &res);
            cudaMemPoolGetAttribute(g->cache->pool, cudaMemPoolAttrUsedMemHigh, &used);
            fprintf(stderr, "[gala] run %.3f ms, pool reserved %.1f MB, used high %.1f MB\n", ms, res / 1e6, used / 1e6);
        }
    } catch (...) {
        wk.release();
        delete g->wk;
        g->wk = nullptr;
        throw;
    }
    g->has_result = true;
}

// ------------------------------------------------------------------ multi-GPU driver (a10)
// §4.3.  Each rank owns vertices [lv0, lv1) of the current level and
// holds them as a global-row CSR; C, Sigma_tot, size and d are replicated.  One
// iteration: prune + decide over the owned vertices (the single-GPU kernels),
// collect the local moves, exchange them sparsely (allgatherv of (v, c) pairs)
// or densely (allgatherv of label slices, then a diff) — chosen by bytes on
// the wire — apply the global move list identically everywhere,
// recompute d' of the owned vertices, and all-reduce the owned sum of
// d' + s with the counters; N and the convergence decision then follow from
// identical integers on every rank.  Phase 2: every rank aggregates its owned
// rows, the partial coarse rows are exchanged and merged, and the coarse graph
// is re-split edge-balanced.
struct DistInfo {
    Comm* comm = nullptr;
    long long v0 = 0, v1 = 0;        // level-0 owned range
    int sync_mode = 0;               // 0 adaptive, 1 dense, 2 sparse
    int backend = 0;                 // 0 fabric (device-resident, peer memory), 1 host-driven NCCL collectives
    long long n_dense = 0, n_sparse = 0;
    double bytes_exchanged = 0;
    // fabric (fabric.cuh): this rank's symmetric region and every rank's mapping of it
    void* region = nullptr;
    std::vector<void*> peers;
    FabDev fab = {};
    bool failed = false;   // a run ended in an error: peers may still touch the region
    bool host_bar = false; // fabric barriers on the host (ranks sharing one device: loopback world > 1)
    // mirror block of the level-0 owned rows: depends only on the graph, built by the first run
    int64_t* m0rp = nullptr;
    int32_t* m0col = nullptr;
    int64_t* m0w = nullptr;
};

// Symmetric region of a rank (cudaMalloc: CUDA IPC needs it), byte offsets:
//   0     arrival counter (ull)          256   epoch (ull, local)      264  error flag (int, local)
//   512   headers [2][FAB_MAXP] ull      1024  scalars [2][FAB_MAXP][FAB_NSCAL] int64
//   4096  inbox [2][istride] int32 (istride = n + 2 world + 2, even)
static void fabric_setup(gala_graph_s* g, DistInfo& di, int64_t n) {
    Comm& cm = *di.comm;
    if (cm.world > FAB_MAXP) { set_err(GALA_E_INVALID, "world > %d", FAB_MAXP); throw GalaError{GALA_E_INVALID}; }
    const long long istride = ((n + 2LL * cm.world + 2) + 1) & ~1LL;
    const size_t bytes = 4096 + sizeof(int32_t) * 2 * (size_t)istride;
    CK(cudaMalloc(&di.region, bytes));
    CK(cudaMemsetAsync(di.region, 0, 4096, g->stream));
    CK(cudaStreamSynchronize(g->stream));
    try {
        di.peers = cm.share_region(di.region, g->stream);   // collective; nobody arrives before all zeroed
    } catch (CommError& e) {
        set_err(GALA_E_NCCL, "%s", e.msg.c_str());
        throw GalaError{GALA_E_NCCL};
    }
    FabDev& f = di.fab;
    f.P = cm.world;
    f.rank = cm.rank;
    for (int r = 0; r < cm.world; ++r) {
        char* b = static_cast<char*>(di.peers[r]);
        f.arrive[r] = reinterpret_cast<ull*>(b);
        f.hdr[r] = reinterpret_cast<ull*>(b + 512);
        f.scal[r] = reinterpret_cast<long long*>(b + 1024);
        f.inbox[r] = reinterpret_cast<int32_t*>(b + 4096);
    }
    f.epoch = reinterpret_cast<ull*>(static_cast<char*>(di.region) + 256);
    f.err = reinterpret_cast<int*>(static_cast<char*>(di.region) + 264);
    f.diag = reinterpret_cast<ull*>(static_cast<char*>(di.region) + 272);
    const char* to = getenv("GALA_FABRIC_TIMEOUT_MS");
    f.timeout_ns = (to && atoll(to) > 0 ? (ull)atoll(to) : 20000ull) * 1000000ull;
    f.istride = istride;
}
static void fabric_release(DistInfo& di) {
    if (!di.region) return;
    if (di.failed) cudaDeviceSynchronize();   // stragglers (loopback: same device) finish first
    if (di.comm) di.comm->release_region(di.peers);
    cudaFree(di.region);
    di.region = nullptr;
}

// Communicators are created once per (uid, rank) and cached for the process
// lifetime: handles built with the same uid share one NCCL communicator, so
// rebuilding a graph (e.g. end-to-end timing) does not re-run ncclCommInitRank.
static Comm* comm_for(const void* uid, int rank, int world, bool loop) {
    static std::mutex mu;
    static std::map<std::string, Comm*> cache;
    std::string key(static_cast<const char*>(uid), 128);
    key += std::to_string(rank) + "/" + std::to_string(world);
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    Comm* c = loop ? static_cast<Comm*>(new LoopComm(uid, rank, world)) : static_cast<Comm*>(new NcclComm(uid, rank, world));
    cache[key] = c;
    return c;
}

static std::vector<size_t> prefix_bytes(const std::vector<size_t>& c) {
    std::vector<size_t> d(c.size(), 0);
    for (size_t i = 1; i < c.size(); ++i) d[i] = d[i - 1] + c[i - 1];
    return d;
}

template <int M, bool UNIT>
static void dist_iteration(gala_graph_s* g, Work& wk, const DevCSR& G, long long lv0, long long lv1,
                           const std::vector<long long>& bounds, typename ModeT<M>::ST qW, typename ModeT<M>::ST p,
                           i128 qW128, i128 T, Timer& tm, int64_t maxdeg, int idbits, bool single, int2* lmoves,
                           int2* gmoves, int32_t* newC, ull* dcnt, int64_t* vec) {
    DistInfo& di = *g->di;
    Comm& cm = *di.comm;
    cudaStream_t st = g->stream;
    const long long n = G.n;
    const int big = g->num_sms * 8;
    VTimer vt(g);
    k_iter_begin<<<1, 128, 0, st>>>(wk.ctr);
    CKL();
    BinThresholds th;
    for (int i = 0; i < NBINS - 1; ++i) th.t[i] = g->bins[i];
    k_prune_bin<typename ModeT<M>::ST><<<grid_for((lv1 - lv0 + PB_IPT - 1) / PB_IPT, PB_BT, big), PB_BT, 0, st>>>(
        (int)lv0, (int)lv1, G.rp, wk.d, wk.dp, wk.C, wk.Sig, wk.size, prune_state(g, wk), qW, p, wk.carry, wk.ctr,
        wk.queues, wk.qcap, th);
    CKL();
    launch_decide<M, UNIT>(g, wk, G, qW, p, tm, maxdeg, idbits, single);
    vt.lap("dist: prune+decide");
    CK(cudaMemsetAsync(dcnt, 0, 2 * sizeof(ull), st));
    k_collect_moves<<<grid_for(lv1 - lv0, 256, big), 256, 0, st>>>(wk.ctr, wk.queues, wk.qcap, wk.nextC, lmoves, dcnt);
    CKL();
    ull mloc = 0;
    CK(cudaMemcpyAsync(&mloc, dcnt, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const std::vector<int64_t> cnts = cm.allgather_host((int64_t)mloc, st);
    vt.lap("dist: collect+count");
    long long total = 0;
    for (int64_t c : cnts) total += c;
    const double sparse_bytes = 8.0 * (double)total, dense_bytes = 4.0 * (double)n;
    const bool sparse = di.sync_mode == 2 || (di.sync_mode == 0 && sparse_bytes < dense_bytes);
    if (sparse) {
        std::vector<size_t> cb(cm.world);
        for (int r = 0; r < cm.world; ++r) cb[r] = (size_t)cnts[r] * sizeof(int2);
        cm.allgatherv(lmoves, gmoves, cb, prefix_bytes(cb), st);
        di.n_sparse++;
        di.bytes_exchanged += sparse_bytes;
    } else {
        k_copy_range<<<grid_for(lv1 - lv0, 256, big), 256, 0, st>>>(lv0, lv1, wk.C, newC);
        CKL();
        k_scatter_moves<<<grid_for((long long)mloc, 256, big), 256, 0, st>>>(lmoves, dcnt, newC);
        CKL();
        std::vector<size_t> cb(cm.world), db(cm.world);
        for (int r = 0; r < cm.world; ++r) {
            cb[r] = (size_t)(bounds[r + 1] - bounds[r]) * sizeof(int32_t);
            db[r] = (size_t)bounds[r] * sizeof(int32_t);
        }
        cm.allgatherv(newC + lv0, newC, cb, db, st);
        k_diff_moves<<<grid_for(n, 256, big), 256, 0, st>>>((int)n, wk.C, newC, gmoves, dcnt + 1);
        CKL();
        di.n_dense++;
        di.bytes_exchanged += dense_bytes;
    }
    vt.lap(sparse ? "dist: exchange sparse" : "dist: exchange dense");
    k_apply_list<<<grid_for(total, 256, big), 256, 0, st>>>(gmoves, total, wk.C, wk.Sig, wk.size, wk.d, wk.stamp,
                                                             wk.carry, wk.ctr);
    CKL();
    // d' of the owned vertices from its definition (edge-parallel over the owned rows)
    k_dp_zero<<<big, 256, 0, st>>>(wk.ctr, (int)lv0, (int)lv1, wk.dp, G.nnz, 0, 1, 2);
    CKL();
    if (G.nnz) {
        k_dp_full<UNIT><<<grid_for((G.nnz + 127) / 128 * 32, 256, big), 256, 0, st>>>(wk.ctr, G.nnz, G.row, G.col, G.w,
                                                                                     wk.C, wk.dp, 0, 1, 2, nullptr, nullptr,
                                                                                     nullptr, nullptr, wk.carry);
        CKL();
    }
    vt.lap("dist: apply+dp");
    k_reduce<256><<<wk.reduce_grid, 256, 0, st>>>((int)n, (int)lv0, (int)lv1, wk.dp, wk.s_live(), wk.Sig, wk.part_dc,
                                                  wk.part_s2, wk.part_min, wk.ctr, wk.carry, 0, 0, 0, 0, 0, 3);
    CKL();
    k_pack_counters<<<1, 32, 0, st>>>(wk.carry, wk.ctr, vec);
    CKL();
    cm.allreduce_sum_i64(vec, 5, st);
    k_finish<<<1, 32, 0, st>>>(vec, wk.ctr, wk.carry, (long long)(qW128 >> 64), (ull)qW128, (long long)p,
                               (long long)(T >> 64), (ull)T, 1);
    CKL();
    k_record<<<1, 32, 0, st>>>(wk.ctr, wk.carry, wk.log, wk.log_cap, g->opt_max_iters, 0ull);
    CKL();
    vt.lap("dist: reduce+allreduce");
}

// merge the partial coarse rows of every rank into the full coarse graph, then keep rows [lo, hi)
static void dist_coarsen(gala_graph_s* g, Work& wk, const DevCSR& cur, int64_t nl, long long k, const int32_t* newid,
                         const int32_t* minmem, bool unit, DevCSR& local, std::vector<long long>& bounds,
                         int64_t& maxdeg, int64_t& dmax) {
    Comm& cm = *g->di->comm;
    cudaStream_t st = g->stream;
    const int big = g->num_sms * 8;
    DevCSR part;
    int64_t md = 0;
    int64_t* snew = dalloc<int64_t>(k, st);
    aggregate_rows(g, cur, nl, k, newid, newid, unit, part, md, snew);
    const std::vector<int64_t> cnts = cm.allgather_host(part.nnz, st);
    long long tot = 0;
    for (int64_t c : cnts) tot += c;
    std::vector<size_t> c4(cm.world), c8(cm.world);
    for (int r = 0; r < cm.world; ++r) { c4[r] = (size_t)cnts[r] * 4; c8[r] = (size_t)cnts[r] * 8; }
    int32_t* arow = dalloc<int32_t>(tot, st);
    int32_t* acol = dalloc<int32_t>(tot, st);
    int64_t* aw = dalloc<int64_t>(tot, st);
    cm.allgatherv(part.row, arow, c4, prefix_bytes(c4), st);
    cm.allgatherv(part.col, acol, c4, prefix_bytes(c4), st);
    cm.allgatherv(part.w, aw, c8, prefix_bytes(c8), st);
    g->di->bytes_exchanged += 16.0 * (double)tot;
    dfree(part.rp, st); dfree(part.col, st); dfree(part.w, st); dfree(part.row, st);
    // counting sort of the triplets by coarse row -> multigraph M, then merge duplicates
    DevCSR mg;
    mg.n = k;
    mg.nnz = tot;
    long long* cnt = dalloc<long long>(k + 1, st);
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (k + 1), st));
    k_count_rows<<<grid_for(tot, 256, big), 256, 0, st>>>(tot, arow, cnt);
    CKL();
    mg.rp = dalloc<int64_t>(k + 1, st);
    scan_excl(cnt, reinterpret_cast<long long*>(mg.rp), k, st);
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (k + 1), st));
    mg.row = dalloc<int32_t>(tot, st);
    mg.col = dalloc<int32_t>(tot, st);
    mg.w = dalloc<int64_t>(tot, st);
    k_scatter_rows<<<grid_for(tot, 256, big), 256, 0, st>>>(tot, arow, acol, aw, reinterpret_cast<long long*>(mg.rp),
                                                            cnt, mg.row, mg.col, mg.w);
    CKL();
    dfree(arow, st); dfree(acol, st); dfree(aw, st); dfree(cnt, st);
    int32_t* id = dalloc<int32_t>(k, st);
    k_iota<<<grid_for(k, 256, big), 256, 0, st>>>(k, id);
    CKL();
    DevCSR full;
    aggregate_rows(g, mg, k, k, id, id, false, full, md, snew);
    dfree(mg.rp, st); dfree(mg.col, st); dfree(mg.w, st); dfree(mg.row, st); dfree(id, st);
    // replicated coarse d = Sigma_tot, s = diagonal
    int64_t* dnew = dalloc<int64_t>(k, st);
    ull* dev_max = dalloc<ull>(1, st);
    CK(cudaMemsetAsync(dev_max, 0, sizeof(ull), st));
    k_coarsen_deg<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, newid, wk.Sig, dnew);
    CKL();
    k_max_i64<<<grid_for(k, 256, big), 256, 0, st>>>(k, dnew, dev_max);
    CKL();
    CK(cudaMemcpyAsync(wk.d, dnew, sizeof(int64_t) * k, cudaMemcpyDeviceToDevice, st));
    CK(cudaMemcpyAsync(wk.s, snew, sizeof(int64_t) * k, cudaMemcpyDeviceToDevice, st));
    wk.s_zero = false;
    // edge-balanced split of the coarse graph; keep this rank's rows
    long long* dbounds = dalloc<long long>(cm.world + 1, st);
    k_partition_bounds<<<1, 64, 0, st>>>(k, full.rp, cm.world, dbounds);
    CKL();
    bounds.assign(cm.world + 1, 0);
    ull hm = 0;
    CK(cudaMemcpyAsync(bounds.data(), dbounds, sizeof(long long) * (cm.world + 1), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&hm, dev_max, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    dmax = (int64_t)hm;
    const long long lo = bounds[cm.rank], hi = bounds[cm.rank + 1];
    int64_t e_lo = 0, e_hi = 0;
    CK(cudaMemcpyAsync(&e_lo, full.rp + lo, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&e_hi, full.rp + hi, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    local.n = k;
    local.nnz = e_hi - e_lo;
    local.rp = dalloc<int64_t>(k + 1, st);
    k_restrict_rp<<<grid_for(k + 1, 256, big), 256, 0, st>>>(k, lo, hi, full.rp, local.rp);
    CKL();
    local.col = dalloc<int32_t>(local.nnz, st);
    local.w = dalloc<int64_t>(local.nnz, st);
    local.row = dalloc<int32_t>(local.nnz, st);
    if (local.nnz) {
        CK(cudaMemcpyAsync(local.col, full.col + e_lo, sizeof(int32_t) * local.nnz, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(local.w, full.w + e_lo, sizeof(int64_t) * local.nnz, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(local.row, full.row + e_lo, sizeof(int32_t) * local.nnz, cudaMemcpyDeviceToDevice, st));
    }
    ull* rmax = dalloc<ull>(1, st);
    CK(cudaMemsetAsync(rmax, 0, sizeof(ull), st));
    k_rowmax<<<grid_for(k, 256, big), 256, 0, st>>>(k, reinterpret_cast<long long*>(local.rp), rmax);
    CKL();
    ull hr = 0;
    CK(cudaMemcpyAsync(&hr, rmax, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    maxdeg = (int64_t)hr;
    dfree(full.rp, st); dfree(full.col, st); dfree(full.w, st); dfree(full.row, st);
    dfree(dnew, st); dfree(dev_max, st); dfree(dbounds, st); dfree(rmax, st); dfree(snew, st);
}

// Phase 2 across ranks, send-to-owner (SURVEY.md §8(e) "Phase 2"): every rank aggregates its
// owned rows into partial coarse rows (the single-GPU aggregation); the next level's coarse
// vertex ranges are cut edge-balanced on the all-reduced partial row lengths (an upper bound of
// the merged lengths, identical on every rank); each partial row goes to its owner only
// (alltoallv), which merges what it received into its own coarse rows.  No rank ever holds the
// whole coarse graph.  Coarse d = Sigma_tot (replicated), s = the merged diagonal (owned rows).
static void dist_coarsen_s2o(gala_graph_s* g, Work& wk, const DevCSR& cur, int64_t nl, long long k,
                             const int32_t* newid, const int32_t* minmem, bool unit, DevCSR& local,
                             std::vector<long long>& bounds, int64_t& maxdeg, int64_t& dmax) {
    Comm& cm = *g->di->comm;
    cudaStream_t st = g->stream;
    const int big = g->num_sms * 8;
    const int P = cm.world;
    DevCSR part;
    int64_t md = 0;
    int64_t* snew = dalloc<int64_t>(k, st);
    aggregate_rows(g, cur, nl, k, newid, newid, unit, part, md, snew);
    // next level's ranges from the summed partial lengths
    long long* plen = dalloc<long long>(k + 1, st);
    k_row_lengths<<<grid_for(k, 256, big), 256, 0, st>>>(k, part.rp, plen);
    CKL();
    cm.allreduce_sum_i64(reinterpret_cast<int64_t*>(plen), (size_t)k, st);
    long long* prp = dalloc<long long>(k + 1, st);
    scan_excl(plen, prp, k, st);
    long long* dbounds = dalloc<long long>(P + 1, st);
    k_partition_bounds<<<1, 64, 0, st>>>(k, reinterpret_cast<const int64_t*>(prp), P, dbounds);
    CKL();
    bounds.assign(P + 1, 0);
    CK(cudaMemcpyAsync(bounds.data(), dbounds, sizeof(long long) * (P + 1), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    dfree(plen, st); dfree(prp, st); dfree(dbounds, st);
    // entries of part destined to every rank (rows [b_p, b_{p+1}) are contiguous), counts matrix
    std::vector<long long> eb(P + 1, 0);
    for (int p = 0; p <= P; ++p)
        CK(cudaMemcpyAsync(&eb[p], part.rp + bounds[p], sizeof(long long), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    int64_t* mat = dalloc<int64_t>((size_t)P * P, st);
    std::vector<int64_t> hm((size_t)P * P, 0);
    for (int p = 0; p < P; ++p) hm[(size_t)cm.rank * P + p] = eb[p + 1] - eb[p];
    CK(cudaMemcpyAsync(mat, hm.data(), sizeof(int64_t) * P * P, cudaMemcpyHostToDevice, st));
    cm.allreduce_sum_i64(mat, (size_t)P * P, st);
    CK(cudaMemcpyAsync(hm.data(), mat, sizeof(int64_t) * P * P, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    dfree(mat, st);
    std::vector<size_t> sc(P), sd(P), rc(P), rd(P);
    long long R = 0;
    for (int p = 0; p < P; ++p) {
        sc[p] = (size_t)(eb[p + 1] - eb[p]);
        sd[p] = (size_t)eb[p];
        rc[p] = (size_t)hm[(size_t)p * P + cm.rank];
        rd[p] = (size_t)R;
        R += (long long)rc[p];
    }
    auto scale = [](std::vector<size_t> v, size_t b) { for (auto& x : v) x *= b; return v; };
    int32_t* arow = dalloc<int32_t>(std::max<long long>(R, 1), st);
    int32_t* acol = dalloc<int32_t>(std::max<long long>(R, 1), st);
    int64_t* aw = dalloc<int64_t>(std::max<long long>(R, 1), st);
    cm.alltoallv(part.row, scale(sc, 4), scale(sd, 4), arow, scale(rc, 4), scale(rd, 4), st);
    cm.alltoallv(part.col, scale(sc, 4), scale(sd, 4), acol, scale(rc, 4), scale(rd, 4), st);
    cm.alltoallv(part.w, scale(sc, 8), scale(sd, 8), aw, scale(rc, 8), scale(rd, 8), st);
    g->di->bytes_exchanged += 16.0 * (double)(R - (long long)rc[cm.rank]);
    dfree(part.rp, st); dfree(part.col, st); dfree(part.w, st); dfree(part.row, st);
    // received triplets (own coarse rows only) -> multigraph in global-row form -> merged rows
    DevCSR mg;
    mg.n = k;
    mg.nnz = R;
    long long* cnt = dalloc<long long>(k + 1, st);
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (k + 1), st));
    k_count_rows<<<grid_for(R, 256, big), 256, 0, st>>>(R, arow, cnt);
    CKL();
    mg.rp = dalloc<int64_t>(k + 1, st);
    scan_excl(cnt, reinterpret_cast<long long*>(mg.rp), k, st);
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (k + 1), st));
    mg.row = dalloc<int32_t>(std::max<long long>(R, 1), st);
    mg.col = dalloc<int32_t>(std::max<long long>(R, 1), st);
    mg.w = dalloc<int64_t>(std::max<long long>(R, 1), st);
    k_scatter_rows<<<grid_for(R, 256, big), 256, 0, st>>>(R, arow, acol, aw, reinterpret_cast<long long*>(mg.rp), cnt,
                                                          mg.row, mg.col, mg.w);
    CKL();
    dfree(arow, st); dfree(acol, st); dfree(aw, st); dfree(cnt, st);
    int32_t* id = dalloc<int32_t>(k, st);
    k_iota<<<grid_for(k, 256, big), 256, 0, st>>>(k, id);
    CKL();
    int64_t* snew2 = dalloc<int64_t>(k, st);
    aggregate_rows(g, mg, k, k, id, id, false, local, maxdeg, snew2);
    dfree(mg.rp, st); dfree(mg.col, st); dfree(mg.w, st); dfree(mg.row, st); dfree(id, st); dfree(snew, st);
    // replicated coarse d = Sigma_tot, s = merged diagonal (owned rows; others 0, never read)
    int64_t* dnew = dalloc<int64_t>(k, st);
    ull* dev_max = dalloc<ull>(1, st);
    CK(cudaMemsetAsync(dev_max, 0, sizeof(ull), st));
    k_coarsen_deg<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, newid, wk.Sig, dnew);
    CKL();
    k_max_i64<<<grid_for(k, 256, big), 256, 0, st>>>(k, dnew, dev_max);
    CKL();
    CK(cudaMemcpyAsync(wk.d, dnew, sizeof(int64_t) * k, cudaMemcpyDeviceToDevice, st));
    CK(cudaMemcpyAsync(wk.s, snew2, sizeof(int64_t) * k, cudaMemcpyDeviceToDevice, st));
    wk.s_zero = false;
    ull hm2 = 0;
    CK(cudaMemcpyAsync(&hm2, dev_max, sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    dmax = (int64_t)hm2;
    dfree(dnew, st); dfree(dev_max, st); dfree(snew2, st);
}

// ------------------------------------------------------------------ multi-GPU, fabric backend
// Per-level device state of the fabric iteration (fabric.cuh): the local move list, the mirror
// block of the owned rows (§8(e)) and the d' work items.
struct DistLevel {
    long long lv0 = 0, lv1 = 0;
    int2* lmoves = nullptr;
    ull* lcount = nullptr;
    int64_t* mrp = nullptr;
    int32_t* mcol = nullptr;
    int64_t* mw = nullptr;
    int32_t *it_v = nullptr, *it_old = nullptr, *it_chunk = nullptr;
    FabDev f = {};
    bool mirror_cached = false;   // level 0: the mirror belongs to DistInfo (kept across runs)
    void release(cudaStream_t st) {
        dfree(lmoves, st); dfree(lcount, st);
        if (!mirror_cached) { dfree(mrp, st); dfree(mcol, st); dfree(mw, st); }
        dfree(it_v, st); dfree(it_old, st); dfree(it_chunk, st);
    }
};

static void dist_level_setup(gala_graph_s* g, const DevCSR& G, const std::vector<long long>& bounds, DistLevel& L) {
    cudaStream_t st = g->stream;
    DistInfo& di = *g->di;
    const int P = di.comm->world, r = di.comm->rank;
    const int big = g->num_sms * 8;
    const long long n = G.n;
    L.lv0 = bounds[r];
    L.lv1 = bounds[r + 1];
    L.f = di.fab;
    for (int s = 0; s <= P; ++s) L.f.bnd[s] = bounds[s];
    for (int s = 0; s < P; ++s) L.f.off[s] = (bounds[s] + 2LL * s) & ~1LL;
    L.f.force_dense = di.sync_mode == 1;
    L.lmoves = dalloc<int2>(std::max<long long>(L.lv1 - L.lv0, 1), st);
    L.lcount = dalloc<ull>(1, st);
    CK(cudaMemsetAsync(L.lcount, 0, sizeof(ull), st));
    // mirror block: owned entries (v, u, w) counting-sorted by u (level 0: built once per handle)
    const bool lvl0 = G.col == g->g0.col;
    if (lvl0 && di.m0rp) {
        L.mrp = di.m0rp; L.mcol = di.m0col; L.mw = di.m0w;
        L.mirror_cached = true;
    } else {
    long long* cnt = dalloc<long long>(n + 1, st);
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (n + 1), st));
    k_mirror_count<<<grid_for(G.nnz, 256, big), 256, 0, st>>>(G.nnz, G.col, cnt);
    CKL();
    L.mrp = dalloc<int64_t>(n + 1, st);
    scan_excl(cnt, reinterpret_cast<long long*>(L.mrp), n, st);
    CK(cudaMemsetAsync(cnt, 0, sizeof(long long) * (n + 1), st));
    L.mcol = dalloc<int32_t>(std::max<long long>(G.nnz, 1), st);
    if (G.w) L.mw = dalloc<int64_t>(std::max<long long>(G.nnz, 1), st);
    k_mirror_scatter<<<grid_for(G.nnz, 256, big), 256, 0, st>>>(G.nnz, G.row, G.col, G.w,
                                                                 reinterpret_cast<long long*>(L.mrp), cnt, L.mcol, L.mw);
    CKL();
    dfree(cnt, st);
    if (lvl0) { di.m0rp = L.mrp; di.m0col = L.mcol; di.m0w = L.mw; L.mirror_cached = true; }
    }
    // d' items: one per global mover with a row here + one per DCH-entry chunk of own / mirror rows
    const size_t icap = (size_t)n + (size_t)(2 * G.nnz / DCH) + (size_t)P + 1;
    L.it_v = dalloc<int32_t>(icap, st);
    L.it_old = dalloc<int32_t>(icap, st);
    L.it_chunk = dalloc<int32_t>(icap, st);
}

// Fabric barrier: the device-side k_fab_barrier when every rank has its own GPU; ranks that
// share one device (loopback test backend) never spin in a kernel on each other -- each syncs
// its stream (its peer stores are complete and visible on the shared device) and they meet on
// the host.  The level loop then runs stepwise (no CUDA graph) for those ranks.
static void fab_barrier(gala_graph_s* g, const DistLevel& L, cudaStream_t st) {
    if (g->di->host_bar) {
        CK(cudaStreamSynchronize(st));
        g->di->comm->host_barrier();
        return;
    }
    k_fab_barrier<<<1, 32, 0, st>>>(L.f);
    CKL();
}

// one device-resident iteration of the fabric backend (see fabric.cuh for the sequence)
template <int M, bool UNIT>
static void dist_iteration_fab(gala_graph_s* g, Work& wk, const DevCSR& G, const DistLevel& L,
                               typename ModeT<M>::ST qW, typename ModeT<M>::ST p, i128 qW128, i128 T, Timer& tm,
                               int64_t maxdeg, int idbits, unsigned long long cond, bool single) {
    cudaStream_t st = g->stream;
    const long long n = G.n, lv0 = L.lv0, lv1 = L.lv1;
    const int big = g->num_sms * 8;
    BinThresholds th;
    for (int i = 0; i < NBINS - 1; ++i) th.t[i] = g->bins[i];
    cudaEvent_t e = tm.begin();
    k_prune_bin<typename ModeT<M>::ST><<<grid_for((lv1 - lv0 + PB_IPT - 1) / PB_IPT, PB_BT, big), PB_BT, 0, st>>>(
        (int)lv0, (int)lv1, G.rp, wk.d, wk.dp, wk.C, wk.Sig, wk.size, prune_state(g, wk), qW, p, wk.carry, wk.ctr,
        wk.queues, wk.qcap, th);
    CKL();
    tm.end(KC_PRUNE, e);
    launch_decide<M, UNIT>(g, wk, G, qW, p, tm, maxdeg, idbits, single);
    e = tm.begin();
    k_collect_moves<<<grid_for(lv1 - lv0, 256, big), 256, 0, st>>>(wk.ctr, wk.queues, wk.qcap, wk.nextC, L.lmoves,
                                                                    L.lcount);
    CKL();
    k_fab_push<<<g->num_sms * 2, 256, 0, st>>>(L.f, L.lmoves, L.lcount, wk.C, wk.carry);
    CKL();
    k_fab_push_fix<<<g->num_sms, 256, 0, st>>>(L.f, L.lmoves, L.lcount, wk.carry);
    CKL();
    fab_barrier(g, L, st);
    tm.end(KC_XCHG, e);
    e = tm.begin();
    k_fab_apply<<<grid_for(n, 256, big), 256, 0, st>>>(L.f, wk.carry, wk.ctr, wk.C, wk.Sig, wk.size, wk.d, wk.stamp,
                                                       wk.dp, G.rp, L.mrp, lv0, lv1, L.it_v, L.it_old, L.it_chunk);
    CKL();
    tm.end(KC_APPLY, e);
    e = tm.begin();
    k_fab_dp_delta<UNIT><<<big, 256, 0, st>>>(wk.ctr, G.rp, G.col, G.w, L.mrp, L.mcol, L.mw, wk.C, L.it_v, L.it_old,
                                              L.it_chunk, wk.stamp, wk.dp, wk.carry, G.nnz, g->opt_delta, lv0, lv1, g->opt_delta_den);
    CKL();
    k_dp_zero<<<big, 256, 0, st>>>(wk.ctr, (int)lv0, (int)lv1, wk.dp, G.nnz, g->opt_delta, 1, g->opt_delta_den);
    CKL();
    if (G.nnz) {
        k_dp_full<UNIT><<<grid_for((G.nnz + 127) / 128 * 32, 256, big), 256, 0, st>>>(
            wk.ctr, G.nnz, G.row, G.col, G.w, wk.C, wk.dp, g->opt_delta, 1, g->opt_delta_den, nullptr, nullptr, nullptr, nullptr,
            wk.carry);
        CKL();
    }
    tm.end(KC_DP, e);
    e = tm.begin();
    k_reduce<256><<<wk.reduce_grid, 256, 0, st>>>((int)n, (int)lv0, (int)lv1, wk.dp, wk.s_live(), wk.Sig, wk.part_dc,
                                                  wk.part_s2, wk.part_min, wk.ctr, wk.carry, 0, 0, 0, 0, 0, 3);
    CKL();
    k_fab_scal<<<1, 32, 0, st>>>(L.f, wk.carry, wk.ctr, L.lcount, 0);
    CKL();
    fab_barrier(g, L, st);
    k_fab_finish<<<1, 32, 0, st>>>(L.f, wk.ctr, wk.carry, L.lcount, (long long)(qW128 >> 64), (ull)qW128, (long long)p,
                                   (long long)(T >> 64), (ull)T, 1, wk.log, wk.log_cap, g->opt_max_iters, cond);
    CKL();
    tm.end(KC_REDUCE, e);
}

// level start on the fabric: singletons, N of the singleton partition from rank-ordered sums
static void dist_level_start_fab(gala_graph_s* g, Work& wk, const DevCSR& G, const DistLevel& L, i128 qW128,
                                 int64_t p) {
    cudaStream_t st = g->stream;
    const long long n = G.n;
    k_reduce<256><<<wk.reduce_grid, 256, 0, st>>>((int)n, (int)L.lv0, (int)L.lv1, wk.dp, wk.s_live(), wk.Sig,
                                                  wk.part_dc, wk.part_s2, wk.part_min, wk.ctr, wk.carry, 0, 0, 0, 0, 0,
                                                  2);
    CKL();
    k_fab_scal<<<1, 32, 0, st>>>(L.f, wk.carry, wk.ctr, L.lcount, 1);
    CKL();
    fab_barrier(g, L, st);
    k_fab_finish<<<1, 32, 0, st>>>(L.f, wk.ctr, wk.carry, L.lcount, (long long)(qW128 >> 64), (ull)qW128, (long long)p,
                                   0, 0, 0, nullptr, 0, 0, 0ull);
    CKL();
}

template <int M, bool UNIT>
static void dist_phase1_fab(gala_graph_s* g, Work& wk, const DevCSR& G, const DistLevel& L, typename ModeT<M>::ST qW,
                            typename ModeT<M>::ST p, i128 qW128, i128 T, Timer& tm, int64_t maxdeg, int idbits,
                            std::vector<IterLog>& out, bool single_ok) {
    block_setup<M, UNIT>(g);
    g->cur_n = G.n;
    // ranks sharing a process (loopback) meet on the host before every launch of fabric work, so
    // no rank's barrier kernel spins while another rank's thread is still in host calls that may
    // wait for the whole (shared) device: graph instantiation, pool growth, pageable copies
    level_loop(
        g, wk, out, single_ok, tm,
        [&](unsigned long long cond, bool single) {
            dist_iteration_fab<M, UNIT>(g, wk, G, L, qW, p, qW128, T, tm, maxdeg, idbits, cond, single);
        },
        [&]() { g->di->comm->host_barrier(); });
}

static void do_run_dist(gala_graph_s* g, double gamma, double tol, int max_levels) {
    PoolScope pool_scope(g->cache);
    cudaStream_t st = g->stream;
    CK(cudaSetDevice(g->device));
    DistInfo& di = *g->di;
    Comm& cm = *di.comm;
    g->has_result = false;
    g->trace.clear();
    g->trace_labels.clear();
    g->levels.clear();
    for (int i = 0; i < KC_COUNT; ++i) { g->kc_ms[i] = 0; g->kc_bytes[i] = 0; g->kc_launches[i] = 0; }
    g->dp_mismatch = 0;
    di.n_dense = di.n_sparse = 0;
    di.bytes_exchanged = 0;
    const long long launches0 = g_launches;
    int64_t p, q;
    gamma_to_pq(gamma, &p, &q);
    g->p = p;
    g->q = q;
    const int64_t n0 = g->n0, W = g->W;
    const int64_t mpq = std::max(p, q);
    if ((long double)mpq * (long double)W * (long double)W >= 0x1p125L) {
        set_err(GALA_E_OVERFLOW, "max(p,q)*W^2 >= 2^125");
        throw GalaError{GALA_E_OVERFLOW};
    }
    const i128 qW128 = (i128)q * W;
    const i128 T = (i128)ceill((long double)tol * (long double)q * (long double)W * (long double)W);
    const int big = g->num_sms * 8;
    if (!g->lab) g->lab = dalloc<int32_t>(n0, st);
    ensure_workspace(g);
    Work& wk = *g->wk;
    CK(cudaEventRecord(wk.ev[0], st));
    int2* lmoves = dalloc<int2>(n0, st);
    int2* gmoves = dalloc<int2>(n0, st);
    int32_t* newC = dalloc<int32_t>(n0, st);
    ull* dcnt = dalloc<ull>(2, st);
    int64_t* vec = dalloc<int64_t>(8, st);
    try {
        CK(cudaMemsetAsync(wk.ctr, 0, sizeof(IterCounters), st));
        CK(cudaMemsetAsync(wk.carry, 0, sizeof(Carry), st));
        DevCSR cur = g->g0;
        bool cur_owned = false;
        CK(cudaMemcpyAsync(wk.d, g->d0, sizeof(int64_t) * n0, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(wk.s, g->s0, sizeof(int64_t) * n0, cudaMemcpyDeviceToDevice, st));
        wk.s_zero = !g->self0;
        int64_t maxdeg = g->maxdeg0, dmax = g->maxw0;
        std::vector<long long> bounds = g->dbounds0;
        Timer tm(g);
        std::vector<IterLog> logs;
        for (int level = 0;; ++level) {
            const int64_t nl = cur.n;
            const bool unit = (cur.w == nullptr);
            const long long lv0 = bounds[cm.rank], lv1 = bounds[cm.rank + 1];
            long long gnnz = 0;   // level nnz over all ranks (stats / nominal edges)
            for (int64_t x : cm.allgather_host(cur.nnz, st)) gnnz += x;
            LevelStat ls{};
            ls.n = nl;
            ls.nnz = gnnz;
            ls.maxdeg = maxdeg;
            CK(cudaEventRecord(wk.ev[2], st));
            if (lv1 - lv0 > wk.qcap) {   // this level's owned range is longer than any before
                dfree(wk.queues, st);
                wk.qcap = lv1 - lv0;
                wk.queues = dalloc<QRec>((size_t)wk.qcap * (NBINS / 2), st);
            }
            prepare_level_tables(g, wk, cur, maxdeg);
            k_level_init<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.d, wk.C, wk.Sig, wk.size, wk.dp, wk.stamp, wk.cst,
                                                                 wk.carry, prune_state(g, wk));
            CKL();
            if (level == 0) CK(cudaMemcpyAsync(g->lab, wk.C, sizeof(int32_t) * n0, cudaMemcpyDeviceToDevice, st));
            k_iter_begin<<<1, 128, 0, st>>>(wk.ctr);
            CKL();
            const bool fab = di.backend == 0;
            DistLevel L;
            if (fab) {
                dist_level_setup(g, cur, bounds, L);
                cm.host_barrier();   // loopback: every rank's host-side level setup done (see dist_phase1_fab)
                dist_level_start_fab(g, wk, cur, L, qW128, p);
            } else {
                k_reduce<256><<<wk.reduce_grid, 256, 0, st>>>((int)nl, (int)lv0, (int)lv1, wk.dp, wk.s_live(), wk.Sig, wk.part_dc,
                                                              wk.part_s2, wk.part_min, wk.ctr, wk.carry, 0, 0, 0, 0, 0, 2);
                CKL();
                k_pack_counters<<<1, 32, 0, st>>>(wk.carry, wk.ctr, vec);
                CKL();
                cm.allreduce_sum_i64(vec, 5, st);
                k_finish<<<1, 32, 0, st>>>(vec, wk.ctr, wk.carry, (long long)(qW128 >> 64), (ull)qW128, (long long)p, 0, 0, 0);
                CKL();
            }
            CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            const i128 N_start = carry_N(wk.h_carry);
            const ull t_level = wk.h_carry->t_ns;
            int idbits = 1;
            while (idbits < 31 && ((int64_t)1 << idbits) < nl) ++idbits;
            const long double bound = (long double)mpq * (long double)W * (long double)std::max<int64_t>(dmax, 1);
            int mode = DM_FAST;
            if (g->opt_force_i128 || bound >= 0x1p62L || dmax >= ((int64_t)1 << 32)) mode = DM_W128;
            else if (bound * (long double)((int64_t)1 << idbits) >= 0x1p62L || g->opt_force_wide)
                mode = DM_W64;
            ls.i128path = mode;
            const long long qW64 = (long long)qW128, p64 = (long long)p;
            logs.clear();
            const bool single_ok = level > 0 || g->rows_distinct0;
            if (fab) {
#define DIST_FAB(MM, UU, QW, PP) dist_phase1_fab<MM, UU>(g, wk, cur, L, QW, PP, qW128, T, tm, maxdeg, idbits, logs, single_ok)
                if (mode == DM_W128) { if (unit) DIST_FAB(DM_W128, true, (i128)qW128, (i128)p); else DIST_FAB(DM_W128, false, (i128)qW128, (i128)p); }
                else if (mode == DM_W64) { if (unit) DIST_FAB(DM_W64, true, qW64, p64); else DIST_FAB(DM_W64, false, qW64, p64); }
                else { if (unit) DIST_FAB(DM_FAST, true, qW64, p64); else DIST_FAB(DM_FAST, false, qW64, p64); }
#undef DIST_FAB
                L.release(st);
                int err = 0;
                ull diag[2] = {0, 0};
                CK(cudaMemcpyAsync(&err, di.fab.err, sizeof(int), cudaMemcpyDeviceToHost, st));
                CK(cudaMemcpyAsync(diag, di.fab.diag, sizeof(diag), cudaMemcpyDeviceToHost, st));
                CK(cudaStreamSynchronize(st));
                if (err) {
                    char msg[256];
                    snprintf(msg, sizeof msg, "fabric: a peer rank stopped answering (rank %d, level %d, barrier %llu, "
                             "arrivals %llu of %llu)", cm.rank, level, diag[0], diag[1], (diag[0] + 1) * (ull)cm.world);
                    throw CommError{msg};
                }
            }
            for (int it = 0; !fab; ++it) {
                const bool single = it == 0 && g->opt_singleton && single_ok;
#define DIST_IT(MM, UU, QW, PP) dist_iteration<MM, UU>(g, wk, cur, lv0, lv1, bounds, QW, PP, qW128, T, tm, maxdeg, \
                                                       idbits, single, lmoves, gmoves, newC, dcnt, vec)
                if (mode == DM_W128) { if (unit) DIST_IT(DM_W128, true, (i128)qW128, (i128)p); else DIST_IT(DM_W128, false, (i128)qW128, (i128)p); }
                else if (mode == DM_W64) { if (unit) DIST_IT(DM_W64, true, qW64, p64); else DIST_IT(DM_W64, false, qW64, p64); }
                else { if (unit) DIST_IT(DM_FAST, true, qW64, p64); else DIST_IT(DM_FAST, false, qW64, p64); }
#undef DIST_IT
                CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
                CK(cudaMemcpyAsync(wk.h_log, wk.log + (it % wk.log_cap), sizeof(IterLog), cudaMemcpyDeviceToHost, st));
                if (g->opt_trace >= 2) {
                    g->trace_labels.emplace_back(nl);
                    CK(cudaMemcpyAsync(g->trace_labels.back().data(), wk.C, sizeof(int32_t) * nl, cudaMemcpyDeviceToHost, st));
                }
                CK(cudaStreamSynchronize(st));
                tm.resolve();
                logs.push_back(*wk.h_log);
                const Carry& c = *wk.h_carry;
                if (!c.more && !c.converged && !(g->opt_max_iters > 0 && c.iter >= g->opt_max_iters)) {
                    int base = c.iter;   // log full: restart slots
                    CK(cudaMemcpyAsync(&wk.carry->log_base, &base, sizeof(int), cudaMemcpyHostToDevice, st));
                }
                if (c.converged || (g->opt_max_iters > 0 && c.iter >= g->opt_max_iters)) break;
            }
            i128 N = N_start;
            ull t_prev = t_level;
            for (size_t it = 0; it < logs.size(); ++it) {
                const IterCounters& c = logs[it].ctr;
                N = log_N(logs[it]);
                int64_t scanned = 0, kk = 0;
                for (int b = 0; b < NBINS; ++b) { scanned += (int64_t)c.bin_deg[b]; kk += (int64_t)c.bin_k[b]; }
                ls.edges_scanned += scanned;
                ls.nominal_edges += gnnz;
                const int64_t it_ns = fab && logs[it].t_ns >= t_prev ? (int64_t)(logs[it].t_ns - t_prev) : 0;
                if (fab) {
                    t_prev = logs[it].t_ns;
                    if (c.n_dense) di.n_dense++; else di.n_sparse++;
                    di.bytes_exchanged += (double)c.xbytes;
                }
                if (g->opt_trace >= 1) {
                    TraceRec r;
                    r.v[0] = level; r.v[1] = (int64_t)it; r.v[2] = nl; r.v[3] = (int64_t)c.n_active;
                    r.v[4] = (int64_t)c.n_pruned; r.v[5] = (int64_t)c.n_moved;
                    r.v[6] = (int64_t)(N >> 64); r.v[7] = (int64_t)(uint64_t)N;
                    r.v[8] = scanned; r.v[9] = kk; r.v[10] = (int64_t)c.delta_used;
                    r.v[11] = fab ? 1 + (int64_t)c.n_dense : 0;   // fabric: 1 + senders that went dense
                    r.v[12] = 0; r.v[13] = (int64_t)c.xbytes; r.v[14] = it_ns; r.v[15] = 0;
                    g->trace.push_back(r);
                }
            }
            ls.iters = (int64_t)logs.size();
            if (fab && !logs.empty()) ls.ms_iters = (double)(logs.back().t_ns - t_level) * 1e-6;
            CK(cudaEventRecord(wk.ev[3], st));
            // a8: relabel (replicated state: identical on every rank)
            int32_t* minmem = dalloc<int32_t>(nl, st);
            long long* pos = dalloc<long long>(nl + 1, st);
            int32_t* newid = dalloc<int32_t>(nl, st);
            k_fill_i32<<<grid_for(nl, 256, big), 256, 0, st>>>(minmem, nl, INT_MAX);
            CKL();
            k_minmember<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem);
            CKL();
            k_minflag<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, pos);
            CKL();
            scan_excl(pos, pos, nl, st);
            k_newid<<<grid_for(nl, 256, big), 256, 0, st>>>((int)nl, wk.C, minmem, pos, newid);
            CKL();
            k_compose<<<grid_for(n0, 256, big), 256, 0, st>>>(n0, newid, g->lab);
            CKL();
            long long kcomm = 0;
            CK(cudaMemcpyAsync(&kcomm, pos + nl, sizeof(long long), cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            g->k_final = kcomm;   // canonical final labels are 0..k-1 (reading c19)
            const bool stop = (kcomm == nl) || (max_levels > 0 && level + 1 >= max_levels) || (N - N_start < T);
            DevCSR nxt;
            if (!stop) {
                if (di.backend == 0) dist_coarsen_s2o(g, wk, cur, nl, kcomm, newid, minmem, unit, nxt, bounds, maxdeg, dmax);
                else dist_coarsen(g, wk, cur, nl, kcomm, newid, minmem, unit, nxt, bounds, maxdeg, dmax);
            }
            dfree(minmem, st);
            dfree(pos, st);
            dfree(newid, st);
            CK(cudaEventRecord(wk.ev[4], st));
            CK(cudaEventSynchronize(wk.ev[4]));
            float ms1 = 0, ms2 = 0;
            CK(cudaEventElapsedTime(&ms1, wk.ev[2], wk.ev[3]));
            CK(cudaEventElapsedTime(&ms2, wk.ev[3], wk.ev[4]));
            ls.ms_phase1 = ms1;
            ls.ms_phase2 = ms2;
            g->levels.push_back(ls);
            if (cur_owned) { dfree(cur.rp, st); dfree(cur.col, st); dfree(cur.w, st); dfree(cur.row, st); }
            if (stop) break;
            cur = nxt;
            cur_owned = true;
        }
        CK(cudaMemcpyAsync(wk.h_carry, wk.carry, sizeof(Carry), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        g->N = carry_N(wk.h_carry);
        g->check_mismatch = 0;
        CK(cudaEventRecord(wk.ev[1], st));
        CK(cudaEventSynchronize(wk.ev[1]));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, wk.ev[0], wk.ev[1]));
        g->run_ms = ms;
        g->launches = g_launches - launches0;
    } catch (CommError& e) {
        cm.abort();
        di.failed = true;
        dfree(lmoves, st); dfree(gmoves, st); dfree(newC, st); dfree(dcnt, st); dfree(vec, st);
        set_err(GALA_E_NCCL, "%s", e.msg.c_str());
        throw GalaError{GALA_E_NCCL};
    } catch (...) {
        cm.abort();   // peers blocked in a collective raise instead of waiting forever
        di.failed = true;
        dfree(lmoves, st); dfree(gmoves, st); dfree(newC, st); dfree(dcnt, st); dfree(vec, st);
        throw;
    }
    dfree(lmoves, st); dfree(gmoves, st); dfree(newC, st); dfree(dcnt, st); dfree(vec, st);
    g->has_result = true;
}

// ------------------------------------------------------------------ creation
static void init_graph_common(gala_graph_s* g, int64_t n, int device, uintptr_t stream) {
    g->device = device;
    CK(cudaSetDevice(device));
    // one attribute query (cudaGetDeviceProperties fills the whole struct: milliseconds per handle)
    CK(cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, device));
    if (stream) {
        g->stream = reinterpret_cast<cudaStream_t>(stream);
        g->own_stream = false;
    } else {
        CK(cudaStreamCreate(&g->stream));   // blocking: ordered after legacy-default-stream work
        g->own_stream = true;
    }
    g->n0 = n;
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = device;
    {
        std::lock_guard<std::mutex> lk(g_stash_mu);
        auto it = g_stash.find(device);
        if (it != g_stash.end()) { g->cache = it->second; g_stash.erase(it); }
    }
    if (!g->cache) {
        g->cache = new DevCache();
        CK(cudaMemPoolCreate(&g->cache->pool, &props));
        uint64_t keep = UINT64_MAX;
        CK(cudaMemPoolSetAttribute(g->cache->pool, cudaMemPoolAttrReleaseThreshold, &keep));
    }
    g_cache = g->cache;
}

// Device-side validation of the copied CSR (GALA_E_INVALID), unit-weight
// detection, d(v), s(v), max row length, max weighted degree, W (int128-checked)
// and the level-0 row-id array.
static void finish_graph(gala_graph_s* g) {
    cudaStream_t st = g->stream;
    const int64_t n = g->n0;
    const int big = g->num_sms * 8;
    unsigned* flags = dalloc<unsigned>(1, st);
    CK(cudaMemsetAsync(flags, 0, sizeof(unsigned), st));
    k_validate<<<grid_for(std::max<int64_t>(n, g->g0.nnz), 256, big), 256, 0, st>>>((int)n, g->g0.nnz, g->g0.rp,
                                                                                   g->g0.col, g->g0.w, flags);
    CKL();
    unsigned hf = 0;
    CK(cudaMemcpyAsync(&hf, flags, sizeof(unsigned), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    dfree(flags, st);
    if (hf & 1u) { set_err(GALA_E_INVALID, "row_ptr not monotone"); throw GalaError{GALA_E_INVALID}; }
    if (hf & 2u) { set_err(GALA_E_INVALID, "col_idx out of range"); throw GalaError{GALA_E_INVALID}; }
    if (hf & 4u) { set_err(GALA_E_INVALID, "weight <= 0"); throw GalaError{GALA_E_INVALID}; }
    if (g->g0.w && !(hf & 8u)) dfree(g->g0.w, st);   // all weights 1: unit-weight level 0
    g->d0 = dalloc<int64_t>(n, st);
    g->s0 = dalloc<int64_t>(n, st);
    g->g0.row = dalloc<int32_t>(g->g0.nnz, st);
    k_fill_rows<<<grid_for(n * 32, 256, big), 256, 0, st>>>((int)n, g->g0.rp, g->g0.row);
    CKL();
    ull* mx = dalloc<ull>(4, st);
    CK(cudaMemsetAsync(mx, 0, 4 * sizeof(ull), st));
    int grid = grid_for(n * 32, 256, big);
    if (g->g0.w == nullptr)
        k_degrees<true><<<grid, 256, 0, st>>>((int)n, g->g0.rp, g->g0.col, g->g0.w, g->d0, g->s0, mx);
    else
        k_degrees<false><<<grid, 256, 0, st>>>((int)n, g->g0.rp, g->g0.col, g->g0.w, g->d0, g->s0, mx);
    CKL();
    k_max_i64<<<grid_for(n, 256, big), 256, 0, st>>>(n, g->d0, mx + 1);
    CKL();
    k_rows_not_increasing<<<grid_for(g->g0.nnz, 256, big), 256, 0, st>>>(g->g0.nnz, g->g0.row, g->g0.col, mx + 2);
    CKL();
    i128* part = dalloc<i128>(big, st);
    ull* ticket = dalloc<ull>(1, st);
    i128* wsum = dalloc<i128>(1, st);
    CK(cudaMemsetAsync(ticket, 0, sizeof(ull), st));
    k_sum_i128<<<grid_for(n, 256, big), 256, 0, st>>>(n, g->d0, part, ticket, wsum);
    CKL();
    ull hm[4];
    i128 hW = 0;
    CK(cudaMemcpyAsync(hm, mx, 4 * sizeof(ull), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&hW, wsum, sizeof(i128), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    g->maxdeg0 = (int64_t)hm[0];
    g->maxw0 = (int64_t)hm[1];
    g->rows_distinct0 = (hm[2] == 0);
    g->self0 = (hm[3] != 0);
    dfree(mx, st);
    dfree(part, st);
    dfree(ticket, st);
    dfree(wsum, st);
    if (n == 0) hW = 0;
    if (hW >= ((i128)1 << 62)) { set_err(GALA_E_OVERFLOW, "total weight W >= 2^62"); throw GalaError{GALA_E_OVERFLOW}; }
    g->W = (int64_t)hW;
    // per-entry neighbour communities (ckey[e] = C[col[e]], rewritten by every full d' pass and
    // invalidated by a delta pass) need no reverse-entry index: single GPU, sorted rows, int32 entry ids
    g->ckey_ok = !g->di && g->rows_distinct0 && g->g0.nnz > 0 && g->g0.nnz < ((int64_t)1 << 31);
}

#define API_BEGIN try {
#define API_END                                              \
    }                                                        \
    catch (GalaError & e_) { return e_.st; }                 \
    catch (std::exception & e_) { return set_err(GALA_E_CUDA, "%s", e_.what()); } \
    catch (...) { return set_err(GALA_E_CUDA, "unknown error"); }                  \
    return GALA_OK;

extern "C" {

gala_status gala_set_allocator(gala_alloc_fn alloc_fn, gala_free_fn free_fn, void* ctx) {
    if ((alloc_fn == nullptr) != (free_fn == nullptr))
        return set_err(GALA_E_INVALID, "gala_set_allocator: alloc and free must both be set or both NULL");
    std::lock_guard<std::mutex> lk(g_ualloc_mu);
    g_ualloc.alloc = alloc_fn;
    g_ualloc.free = free_fn;
    g_ualloc.ctx = alloc_fn ? ctx : nullptr;
    return GALA_OK;
}

const char* gala_version(void) { return GALA_VERSION; }
const char* gala_last_error(void) { return g_err.c_str(); }

gala_status gala_graph_from_csr(int64_t n, const int64_t* row_ptr, const int32_t* col_idx, const int64_t* weights,
                                int device, uintptr_t stream, gala_graph* out) {
    if (!out) return set_err(GALA_E_INVALID, "out is NULL");
    *out = nullptr;
    if (n < 0 || n >= ((int64_t)1 << 31)) return set_err(GALA_E_INVALID, "n out of range: %lld", (long long)n);
    if (!row_ptr) return set_err(GALA_E_INVALID, "row_ptr is NULL");
    if (row_ptr[0] != 0 || row_ptr[n] < 0) return set_err(GALA_E_INVALID, "row_ptr[0] != 0 or row_ptr[n] < 0");
    if (row_ptr[n] > 0 && !col_idx) return set_err(GALA_E_INVALID, "col_idx is NULL");
    gala_graph_s* g = new gala_graph_s();
    PoolScope pool_scope(nullptr);
    API_BEGIN
    try {
        init_graph_common(g, n, device, stream);
        cudaStream_t st = g->stream;
        const int64_t nnz = row_ptr[n];
        g->nnz0 = nnz;
        g->g0.n = n;
        g->g0.nnz = nnz;
        g->g0.rp = dalloc<int64_t>(n + 1, st);
        g->g0.col = dalloc<int32_t>(nnz, st);
        CK(cudaMemcpyAsync(g->g0.rp, row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, st));
        if (nnz) CK(cudaMemcpyAsync(g->g0.col, col_idx, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, st));
        if (weights) {
            g->g0.w = dalloc<int64_t>(nnz, st);
            CK(cudaMemcpyAsync(g->g0.w, weights, sizeof(int64_t) * nnz, cudaMemcpyHostToDevice, st));
        }
        finish_graph(g);
    } catch (...) {
        gala_graph_free(g);
        throw;
    }
    *out = g;
    API_END
}

gala_status gala_graph_from_csr_device(int64_t n, const int64_t* d_row_ptr, const int32_t* d_col_idx,
                                       const int64_t* d_weights, int device, uintptr_t stream, gala_graph* out) {
    if (!out) return set_err(GALA_E_INVALID, "out is NULL");
    *out = nullptr;
    if (n < 0 || n >= ((int64_t)1 << 31)) return set_err(GALA_E_INVALID, "n out of range");
    gala_graph_s* g = new gala_graph_s();
    PoolScope pool_scope(nullptr);
    API_BEGIN
    try {
        init_graph_common(g, n, device, stream);
        cudaStream_t st = g->stream;
        int64_t nnz = 0, rp0 = 0;
        CK(cudaMemcpyAsync(&nnz, d_row_ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(&rp0, d_row_ptr, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        if (rp0 != 0 || nnz < 0) { set_err(GALA_E_INVALID, "row_ptr[0] != 0"); throw GalaError{GALA_E_INVALID}; }
        g->nnz0 = nnz;
        g->g0.n = n;
        g->g0.nnz = nnz;
        g->g0.rp = dalloc<int64_t>(n + 1, st);
        g->g0.col = dalloc<int32_t>(nnz, st);
        CK(cudaMemcpyAsync(g->g0.rp, d_row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToDevice, st));
        if (nnz) CK(cudaMemcpyAsync(g->g0.col, d_col_idx, sizeof(int32_t) * nnz, cudaMemcpyDeviceToDevice, st));
        if (d_weights) {
            g->g0.w = dalloc<int64_t>(nnz, st);
            CK(cudaMemcpyAsync(g->g0.w, d_weights, sizeof(int64_t) * nnz, cudaMemcpyDeviceToDevice, st));
        }
        finish_graph(g);
    } catch (...) {
        gala_graph_free(g);
        throw;
    }
    *out = g;
    API_END
}

gala_status gala_validate(gala_graph g) {
    if (!g) return set_err(GALA_E_INVALID, "null handle");
    API_BEGIN
    // symmetric check on the host copy (O(nnz log nnz)); debugging aid
    cudaStream_t st = g->stream;
    std::vector<int64_t> rp(g->n0 + 1);
    std::vector<int32_t> col(g->nnz0);
    std::vector<int64_t> w;
    CK(cudaMemcpyAsync(rp.data(), g->g0.rp, sizeof(int64_t) * (g->n0 + 1), cudaMemcpyDeviceToHost, st));
    if (g->nnz0) CK(cudaMemcpyAsync(col.data(), g->g0.col, sizeof(int32_t) * g->nnz0, cudaMemcpyDeviceToHost, st));
    if (g->g0.w) {
        w.resize(g->nnz0);
        CK(cudaMemcpyAsync(w.data(), g->g0.w, sizeof(int64_t) * g->nnz0, cudaMemcpyDeviceToHost, st));
    }
    CK(cudaStreamSynchronize(st));
    std::vector<std::tuple<int32_t, int32_t, int64_t>> a, b;
    a.reserve(g->nnz0);
    b.reserve(g->nnz0);
    for (int64_t v = 0; v < g->n0; ++v)
        for (int64_t e = rp[v]; e < rp[v + 1]; ++e) {
            int64_t x = w.empty() ? 1 : w[e];
            a.emplace_back((int32_t)v, col[e], x);
            b.emplace_back(col[e], (int32_t)v, x);
        }
    std::sort(a.begin(), a.end());
    std::sort(b.begin(), b.end());
    if (a != b) return set_err(GALA_E_INVALID, "CSR is not symmetric");
    API_END
}

gala_status gala_run(gala_graph g, double gamma, double tol, int32_t max_levels) {
    if (g && g->di && (g->opt_prune > 1 || g->opt_prune_check))
        return set_err(GALA_E_INVALID, "prune strategies 2-4 and prune_check are single-GPU only");
    if (!g) return set_err(GALA_E_INVALID, "null handle");
    if (!(gamma > 0) || !(gamma < 1e12)) return set_err(GALA_E_INVALID, "gamma must be > 0");
    if (!(tol > 0)) return set_err(GALA_E_INVALID, "tol must be > 0");
    for (int i = 1; i < NBINS - 1; ++i)
        if (g->bins[i] < g->bins[i - 1]) return set_err(GALA_E_INVALID, "bin thresholds must be non-decreasing");
    API_BEGIN
    if (g->W == 0) {
        // reading c18: no edges -> singletons, Q := 0
        CK(cudaSetDevice(g->device));
        if (!g->lab) g->lab = dalloc<int32_t>(std::max<int64_t>(g->n0, 1), g->stream);
        std::vector<int32_t> iota(g->n0);
        for (int64_t v = 0; v < g->n0; ++v) iota[v] = (int32_t)v;
        if (g->n0) CK(cudaMemcpyAsync(g->lab, iota.data(), sizeof(int32_t) * g->n0, cudaMemcpyHostToDevice, g->stream));
        CK(cudaStreamSynchronize(g->stream));
        gamma_to_pq(gamma, &g->p, &g->q);
        g->N = 0;
        g->k_final = g->n0;
        g->levels.clear();
        g->trace.clear();
        g->trace_labels.clear();
        g->has_result = true;
        return GALA_OK;
    }
    if (g->di) do_run_dist(g, gamma, tol, max_levels);
    else do_run(g, gamma, tol, max_levels);
    API_END
}

static gala_status fetch_labels(gala_graph g, int32_t* out, int64_t n, int64_t* k, bool device) {
    if (!g) return set_err(GALA_E_INVALID, "null handle");
    if (!g->has_result) return set_err(GALA_E_STATE, "gala_run has not completed");
    if (n != g->n0) return set_err(GALA_E_INVALID, "n mismatch (%lld != %lld)", (long long)n, (long long)g->n0);
    API_BEGIN
    CK(cudaSetDevice(g->device));
    std::vector<int32_t> h;
    int32_t* dst = out;
    if (!device) dst = out;
    if (n) CK(cudaMemcpyAsync(dst, g->lab, sizeof(int32_t) * n, device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                              g->stream));
    CK(cudaStreamSynchronize(g->stream));
    if (k && g->k_final >= 0) {   // known from the run's last relabel: no host pass over the labels
        *k = g->k_final;
    } else if (k) {
        if (device) {
            h.resize(n);
            if (n) CK(cudaMemcpy(h.data(), g->lab, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
            dst = h.data();
        }
        int64_t mx = -1;
        for (int64_t v = 0; v < n; ++v) mx = std::max<int64_t>(mx, dst[v]);
        *k = mx + 1;
    }
    API_END
}

gala_status gala_get_communities(gala_graph g, int32_t* labels, int64_t n, int64_t* num_communities) {
    return fetch_labels(g, labels, n, num_communities, false);
}
gala_status gala_get_communities_device(gala_graph g, int32_t* d_labels, int64_t n, int64_t* num_communities) {
    return fetch_labels(g, d_labels, n, num_communities, true);
}

gala_status gala_modularity_numerator(gala_graph g, int64_t* n_hi, uint64_t* n_lo, int64_t* W, int64_t* p, int64_t* q) {
    if (!g) return set_err(GALA_E_INVALID, "null handle");
    if (!g->has_result) return set_err(GALA_E_STATE, "gala_run has not completed");
    if (n_hi) *n_hi = (int64_t)(g->N >> 64);
    if (n_lo) *n_lo = (uint64_t)g->N;
    if (W) *W = g->W;
    if (p) *p = g->p;
    if (q) *q = g->q;
    return GALA_OK;
}

gala_status gala_modularity(gala_graph g, double* q) {
    if (!g || !q) return set_err(GALA_E_INVALID, "null argument");
    if (!g->has_result) return set_err(GALA_E_STATE, "gala_run has not completed");
    if (g->W == 0) { *q = 0.0; return GALA_OK; }
    *q = (double)((long double)g->N / ((long double)g->q * (long double)g->W * (long double)g->W));
    return GALA_OK;
}

void gala_graph_free(gala_graph g) {
    if (!g) return;
    cudaSetDevice(g->device);
    DevCache* const mine = g->cache;
    PoolScope pool_scope(g->cache);
    const bool dist = g->di != nullptr;
    if (g->di) {   // communicators are cached (comm_for); the fabric region is this handle's
        if (g->stream) cudaStreamSynchronize(g->stream);
        fabric_release(*g->di);
        if (g->stream) { dfree(g->di->m0rp, g->stream); dfree(g->di->m0col, g->stream); dfree(g->di->m0w, g->stream); }
        delete g->di;
        g->di = nullptr;
    }
    // GALA_DEBUG_FREE=1: host time of each teardown step on stderr (e2e create/run/free cycles)
    static const bool dbg = getenv("GALA_DEBUG_FREE") != nullptr;
    auto t_prev = std::chrono::steady_clock::now();
    auto lap = [&](const char* what) {
        if (!dbg) return;
        const auto t = std::chrono::steady_clock::now();
        fprintf(stderr, "[gala free] %-10s %8.3f ms\n", what, std::chrono::duration<double, std::milli>(t - t_prev).count());
        t_prev = t;
    };
    cudaStream_t st = g->stream;
    if (g->wk) { g->wk->release(); delete g->wk; g->wk = nullptr; }
    lap("workspace");
    if (st) {
        dfree(g->g0.rp, st);
        dfree(g->g0.col, st);
        dfree(g->g0.w, st);
        dfree(g->g0.row, st);
        dfree(g->d0, st);
        dfree(g->s0, st);
        dfree(g->lab, st);
        cudaStreamSynchronize(st);
        lap("graph+sync");
        // park the idle cache for the next handle on this device (not when it holds blocks of a
        // user allocator: those go back to their owner now)
        if (g->cache && !dist && !cache_has_user_blocks(g->cache) && cudaGetLastError() == cudaSuccess) {
            std::lock_guard<std::mutex> lk(g_stash_mu);
            if (!g_stash.count(g->device)) {
                g_stash[g->device] = g->cache;
                g->cache = nullptr;
            }
        }
        lap(g->cache ? "not parked" : "parked");
        if (g->cache) g->cache->trim(st);
        cudaStreamSynchronize(st);
        if (g->own_stream) cudaStreamDestroy(st);
        lap("trim");
    }
    for (int i = 0; i < 4; ++i) {
        if (g->side[i]) cudaStreamDestroy(g->side[i]);
        if (g->ev_join[i]) cudaEventDestroy(g->ev_join[i]);
    }
    if (g->ev_fork) cudaEventDestroy(g->ev_fork);
    lap("streams");
    if (g->cache) {
        if (g->cache->pool) cudaMemPoolDestroy(g->cache->pool);
        delete g->cache;
    }
    lap("pool");
    g_cache = pool_scope.prev == mine ? nullptr : pool_scope.prev;
    pool_scope.prev = g_cache;
    delete g;
}

gala_status gala_set_option(gala_graph g, const char* key, int64_t value) {
    if (!g || !key) return set_err(GALA_E_INVALID, "null argument");
    PoolScope pool_scope(g->cache);
    std::string k(key);
    if (k == "prune") {
        if (value < 0 || value > 4) return set_err(GALA_E_INVALID, "prune: 0 none, 1 MG, 2 SM, 3 RM, 4 MG+RM");
        g->opt_prune = (int)value;
    } else if (k == "prune_check") g->opt_prune_check = value != 0;
    else if (k == "trace") g->opt_trace = (int)value;
    else if (k == "check") g->opt_check = value != 0;
    else if (k == "timing") g->opt_timing = value != 0;
    else if (k == "max_iters") { if (value < 0) return set_err(GALA_E_INVALID, "max_iters < 0"); g->opt_max_iters = (int)value; }
    else if (k == "delta_den") { if (value < 1 || value > 64) return set_err(GALA_E_INVALID, "delta_den in 1..64"); g->opt_delta_den = (int)value; }
    else if (k == "delta_update") { if (value < 0 || value > 2) return set_err(GALA_E_INVALID, "delta_update in 0..2"); g->opt_delta = (int)value; }
    else if (k == "force_i128") g->opt_force_i128 = value != 0;
    else if (k == "force_wide") {   // 1: DM_W64 everywhere; 2: DM_W64 levels, packed short-row bins
        if (value < 0 || value > 2) return set_err(GALA_E_INVALID, "force_wide in 0..2");
        g->opt_force_wide = (int)value;
    }
    else if (k == "singleton") g->opt_singleton = value != 0;
    else if (k == "agg_big_chunk") g->opt_agg_big_chunk = value != 0;
    else if (k == "agg_chunk") {   // test hook: entries per big-community chunk (1..AGG_CH)
        if (value < 1 || value > AGG_CH) return set_err(GALA_E_INVALID, "agg_chunk must be in [1, 4096]");
        g->opt_agg_chunk = (int)value;
    } else if (k == "agg_bound") {   // phase 2: size big-community tables from chunk distinct counts
        g->opt_agg_bound = value != 0;
    } else if (k == "bin_packed") {   // DM_W64 unit levels: packed argmax keys for rows <= bin_warp512
        g->opt_bin_packed = value != 0;
    } else if (k == "agg_spill") {   // phase 2: spilling block class for segments <= agg_big_ent entries
        g->opt_agg_spill = value != 0;
    } else if (k == "l2_window") {   // persisting-L2 access-policy window on the label array
        g->opt_l2_window = value != 0;
    } else if (k == "table_mode") {   // block-bin hash table (§4.2 ablation): 0 hierarchical, 1 global-only, 2 unified
        if (value < 0 || value > 2) return set_err(GALA_E_INVALID, "table_mode: 0 hierarchical, 1 global-only, 2 unified");
        g->opt_table_mode = (int)value;
    } else if (k == "agg_dense") {   // phase 2: dense k x k accumulation (0 never, 1 auto, 2 whenever k fits)
        if (value < 0 || value > 2) return set_err(GALA_E_INVALID, "agg_dense in 0..2");
        g->opt_agg_dense = (int)value;
    } else if (k == "block_split") {   // block bin: rows <= split in small blocks (0: one class)
        if (value < 0 || value > (1 << 20)) return set_err(GALA_E_INVALID, "block_split must be in [0, 2^20]");
        g->opt_block_split = (int)value;
    } else if (k == "agg_big_ent") {   // phase 2: communities with more entries take the chunked path
        if (value < 1) return set_err(GALA_E_INVALID, "agg_big_ent must be >= 1");
        g->opt_agg_big_ent = value;
    } else if (k == "agg_scap") {  // test hook: block-path smem table cap (512..8192 slots)
        if (value < 512 || value > 8192) return set_err(GALA_E_INVALID, "agg_scap must be in [512, 8192]");
        g->opt_agg_scap = (int)value;
    }
    else if (k == "ckey") g->opt_ckey = value != 0;
    else if (k == "hub_cluster") g->opt_hub_cluster = value != 0;   // hubs on a thread-block cluster (DSMEM tables)
    else if (k == "concurrent") g->opt_concurrent = value != 0;
    else if (k == "verbose") g->opt_verbose = (int)value;
    else if (k == "cuda_graph") g->opt_cuda_graph = value != 0;
    else if (k == "log_cap") { if (value < 2 || value > (1 << 20)) return set_err(GALA_E_INVALID, "log_cap in [2, 2^20]"); g->opt_log_cap = (int)value; }
    else if (k == "hub_smem_slots") {
        if (value < 64 || value > 16384 || (value & (value - 1))) return set_err(GALA_E_INVALID, "hub_smem_slots: power of two in [64, 16384]");
        g->hub_smem_slots = (int)value;
        if (g->wk) { g->wk->release(); delete g->wk; g->wk = nullptr; }
    } else if (k.rfind("bin_", 0) == 0) {
        static const char* names[NBINS - 1] = {"bin_sub4", "bin_sub8", "bin_sub16", "bin_sub32", "bin_warp",
                                               "bin_warp512", "bin_block"};
        static const int lanes[NBINS - 1] = {4, 8, 16, 32, 128, 512, 1 << 30};
        int idx = -1;
        for (int i = 0; i < NBINS - 1; ++i) if (k == names[i]) idx = i;
        if (idx < 0) return set_err(GALA_E_INVALID, "unknown option %s", key);
        if (value < 0 || value > lanes[idx]) return set_err(GALA_E_INVALID, "%s must be in [0, %d]", key, lanes[idx]);
        g->bins[idx] = (int)value;   // monotonicity is checked by gala_run
    } else if (k == "sync_mode") {
        if (value < 0 || value > 2) return set_err(GALA_E_INVALID, "sync_mode: 0 adaptive, 1 dense, 2 sparse");
        g->sync_mode = (int)value;
        if (g->di) g->di->sync_mode = (int)value;
    } else if (k == "dist_backend") {
        if (value < 0 || value > 1) return set_err(GALA_E_INVALID, "dist_backend: 0 fabric (peer memory), 1 host-driven NCCL");
        if (g->di) g->di->backend = (int)value;
    } else return set_err(GALA_E_INVALID, "unknown option %s", key);
    return GALA_OK;
}

gala_status gala_get_trace_count(gala_graph g, int64_t* count) {
    if (!g || !count) return set_err(GALA_E_INVALID, "null argument");
    *count = (int64_t)g->trace.size();
    return GALA_OK;
}
gala_status gala_get_trace_record(gala_graph g, int64_t i, int64_t* out16) {
    if (!g || !out16) return set_err(GALA_E_INVALID, "null argument");
    if (i < 0 || i >= (int64_t)g->trace.size()) return set_err(GALA_E_INVALID, "record index out of range");
    memcpy(out16, g->trace[i].v, sizeof(int64_t) * 16);
    return GALA_OK;
}
gala_status gala_get_trace_labels(gala_graph g, int64_t i, int32_t* out, int64_t n_level) {
    if (!g || !out) return set_err(GALA_E_INVALID, "null argument");
    if (i < 0 || i >= (int64_t)g->trace_labels.size()) return set_err(GALA_E_INVALID, "no labels for record (trace < 2?)");
    if ((int64_t)g->trace_labels[i].size() != n_level) return set_err(GALA_E_INVALID, "n_level mismatch");
    memcpy(out, g->trace_labels[i].data(), sizeof(int32_t) * n_level);
    return GALA_OK;
}

gala_status gala_get_kernel_stats(gala_graph g, int32_t k, const char** name, int64_t* launches, double* ms,
                                  double* alg_bytes, int32_t* count) {
    if (!g) return set_err(GALA_E_INVALID, "null handle");
    if (count) *count = KC_COUNT;
    if (k < 0 || k >= KC_COUNT) return GALA_OK;
    if (name) *name = kc_names[k];
    if (launches) *launches = g->kc_launches[k];
    if (ms) *ms = g->kc_ms[k];
    if (alg_bytes) *alg_bytes = g->kc_bytes[k];
    return GALA_OK;
}

gala_status gala_get_stats(gala_graph g, char* buf, int64_t cap, int64_t* needed) {
    if (!g) return set_err(GALA_E_INVALID, "null handle");
    std::string s = "{";
    char tmp[512];
    snprintf(tmp, sizeof tmp, "\"n\":%lld,\"nnz\":%lld,\"W\":%lld,\"p\":%lld,\"q\":%lld,\"run_ms\":%.6f,\"dp_mismatch\":%lld,"
             "\"kernel_launches\":%lld,\"check_mismatch\":%d,",
             (long long)g->n0, (long long)g->nnz0, (long long)g->W, (long long)g->p, (long long)g->q, g->run_ms,
             (long long)g->dp_mismatch, g->launches, g->check_mismatch);
    s += tmp;
    snprintf(tmp, sizeof tmp, "\"table\":{\"h0_access\":%.0f,\"h1_access\":%.0f,\"h0_keys\":%.0f,\"h1_keys\":%.0f},",
             g->tbl[0], g->tbl[1], g->tbl[2], g->tbl[3]);
    s += tmp;
    if (g->di) {
        snprintf(tmp, sizeof tmp, "\"dist\":{\"rank\":%d,\"world\":%d,\"v0\":%lld,\"v1\":%lld,\"dense_iters\":%lld,"
                 "\"sparse_iters\":%lld,\"bytes_exchanged\":%.0f},",
                 g->di->comm->rank, g->di->comm->world, g->di->v0, g->di->v1, g->di->n_dense, g->di->n_sparse,
                 g->di->bytes_exchanged);
        s += tmp;
    }
    s += "\"levels\":[";
    for (size_t i = 0; i < g->levels.size(); ++i) {
        const LevelStat& l = g->levels[i];
        snprintf(tmp, sizeof tmp,
                 "%s{\"n\":%lld,\"nnz\":%lld,\"iters\":%lld,\"maxdeg\":%lld,\"mode\":%d,\"ms_phase1\":%.6f,"
                 "\"ms_phase2\":%.6f,\"edges_scanned\":%lld,\"nominal_edges\":%lld,\"alg_bytes\":%.0f,\"ms_iters\":%.6f}",
                 i ? "," : "", (long long)l.n, (long long)l.nnz, (long long)l.iters, (long long)l.maxdeg, l.i128path,
                 l.ms_phase1, l.ms_phase2, (long long)l.edges_scanned, (long long)l.nominal_edges, l.alg_bytes,
                 l.ms_iters);
        s += tmp;
    }
    s += "],\"kernels\":{";
    for (int i = 0; i < KC_COUNT; ++i) {
        snprintf(tmp, sizeof tmp, "%s\"%s\":{\"launches\":%lld,\"ms\":%.6f,\"alg_bytes\":%.0f}", i ? "," : "", kc_names[i],
                 (long long)g->kc_launches[i], g->kc_ms[i], g->kc_bytes[i]);
        s += tmp;
    }
    s += "}}";
    if (needed) *needed = (int64_t)s.size() + 1;
    if (!buf || cap < (int64_t)s.size() + 1) return set_err(GALA_E_INVALID, "buffer too small");
    memcpy(buf, s.c_str(), s.size() + 1);
    return GALA_OK;
}

gala_status gala_partition_ranges(int64_t n, const int64_t* row_ptr, int world, int64_t* bounds) {
    if (!row_ptr || !bounds || world < 1 || n < 0) return set_err(GALA_E_INVALID, "bad arguments");
    const int64_t nnz = row_ptr[n];
    bounds[0] = 0;
    int64_t v = 0;
    for (int r = 1; r < world; ++r) {
        // smallest v with row_ptr[v] >= r * nnz / world (edge-balanced), never behind the previous bound
        const long double target = (long double)nnz * r / world;
        int64_t lo = v, hi = n;
        while (lo < hi) {
            int64_t mid = (lo + hi) / 2;
            if ((long double)row_ptr[mid] < target) lo = mid + 1; else hi = mid;
        }
        v = lo;
        bounds[r] = v;
    }
    bounds[world] = n;
    return GALA_OK;
}

gala_status gala_nmi_device(const int32_t* d_x, const int32_t* d_y, int64_t n, int device, uintptr_t stream,
                            double* out) {
    if (!out || n < 0 || (n > 0 && (!d_x || !d_y))) return set_err(GALA_E_INVALID, "null argument or n < 0");
    if (n >= ((int64_t)1 << 31)) return set_err(GALA_E_INVALID, "n >= 2^31");
    if (n == 0) { *out = 1.0; return GALA_OK; }
    API_BEGIN
    CK(cudaSetDevice(device));
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    long long cap = 64;
    while (cap < 2 * n) cap <<= 1;
    unsigned* hist = nullptr;
    ull* keys = nullptr;
    unsigned* cnt = nullptr;
    double* part = nullptr;
    int* bad = nullptr;
    CK(cudaMallocAsync(&hist, sizeof(unsigned) * 2 * (size_t)n, st));
    CK(cudaMallocAsync(&keys, sizeof(ull) * (size_t)cap, st));
    CK(cudaMallocAsync(&cnt, sizeof(unsigned) * (size_t)cap, st));
    CK(cudaMallocAsync(&part, sizeof(double) * (3 * NMI_GRID + 1), st));
    CK(cudaMallocAsync(&bad, sizeof(int), st));
    CK(cudaMemsetAsync(hist, 0, sizeof(unsigned) * 2 * (size_t)n, st));
    CK(cudaMemsetAsync(keys, 0xff, sizeof(ull) * (size_t)cap, st));
    CK(cudaMemsetAsync(cnt, 0, sizeof(unsigned) * (size_t)cap, st));
    CK(cudaMemsetAsync(bad, 0, sizeof(int), st));
    k_nmi_count<<<NMI_GRID, NMI_BT, 0, st>>>(n, d_x, d_y, hist, hist + n, keys, cnt, (ull)(cap - 1), bad);
    CKL();
    k_nmi_terms<<<NMI_GRID, NMI_BT, 0, st>>>(n, hist, hist + n, keys, cnt, cap, part);
    CKL();
    k_nmi_final<<<1, 32, 0, st>>>(part, NMI_GRID, part + 3 * NMI_GRID);
    CKL();
    int hbad = 0;
    double res = 0;
    CK(cudaMemcpyAsync(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&res, part + 3 * NMI_GRID, sizeof(double), cudaMemcpyDeviceToHost, st));
    CK(cudaFreeAsync(hist, st));
    CK(cudaFreeAsync(keys, st));
    CK(cudaFreeAsync(cnt, st));
    CK(cudaFreeAsync(part, st));
    CK(cudaFreeAsync(bad, st));
    CK(cudaStreamSynchronize(st));
    if (hbad) return set_err(GALA_E_INVALID, "gala_nmi_device: a label outside [0, n)");
    *out = res;
    API_END
}

gala_status gala_nccl_unique_id(void* out128) {
    if (!out128) return set_err(GALA_E_INVALID, "null argument");
    if (!nccl_api().load()) return set_err(GALA_E_NCCL, "libnccl.so.2 could not be loaded");
    ncclUniqueId id;
    ncclResult_t r = nccl_api().GetUniqueId(&id);
    if (r != ncclSuccess) return set_err(GALA_E_NCCL, "ncclGetUniqueId: %s", nccl_api().GetErrorString(r));
    memset(out128, 0, 128);
    memcpy(out128, &id, sizeof(id) < 128 ? sizeof(id) : 128);
    return GALA_OK;
}

gala_status gala_loopback_unique_id(void* out128) {
    if (!out128) return set_err(GALA_E_INVALID, "null argument");
    static std::atomic<unsigned long long> counter{0};
    memset(out128, 0, 128);
    const unsigned long long c = ++counter;
    memcpy(out128, "GALALOOP", 8);
    memcpy(static_cast<char*>(out128) + 8, &c, sizeof(c));
    return GALA_OK;
}

gala_status gala_graph_from_csr_dist(const void* uid128, int rank, int world, int device, int64_t n_global,
                                     int64_t v_begin, int64_t v_end, const int64_t* local_row_ptr,
                                     const int32_t* col_idx, const int64_t* weights, uintptr_t stream,
                                     gala_graph* out) {
    if (!out || !uid128 || !local_row_ptr) return set_err(GALA_E_INVALID, "null argument");
    *out = nullptr;
    if (world < 1 || rank < 0 || rank >= world) return set_err(GALA_E_INVALID, "bad rank/world");
    if (n_global < 0 || n_global >= ((int64_t)1 << 31)) return set_err(GALA_E_INVALID, "n out of range");
    if (v_begin < 0 || v_end < v_begin || v_end > n_global) return set_err(GALA_E_INVALID, "bad owned range");
    const int64_t n_own = v_end - v_begin;
    if (local_row_ptr[0] != 0 || local_row_ptr[n_own] < 0) return set_err(GALA_E_INVALID, "local row_ptr[0] != 0");
    const bool loop = memcmp(uid128, "GALALOOP", 8) == 0;
    if (loop && world > 1) {
        // loopback ranks share one CUDA context: a kernel loaded lazily on first use waits for the
        // context to go idle, which another rank's long-running work on the shared device can
        // delay indefinitely (the fabric meets on the host for these ranks, see fab_barrier)
        const char* ml = getenv("CUDA_MODULE_LOADING");
        if (!ml || strcmp(ml, "EAGER") != 0)
            return set_err(GALA_E_INVALID, "loopback with world > 1 needs CUDA_MODULE_LOADING=EAGER (set before CUDA starts)");
    }
    if (!loop && !nccl_api().load()) return set_err(GALA_E_NCCL, "libnccl.so.2 could not be loaded");
    gala_graph_s* g = new gala_graph_s();
    PoolScope pool_scope(nullptr);
    API_BEGIN
    try {
        init_graph_common(g, n_global, device, stream);
        cudaStream_t st = g->stream;
        g->di = new DistInfo();
        try {
            g->di->comm = comm_for(uid128, rank, world, loop);
            g->di->host_bar = !g->di->comm->device_barrier_ok();
            g->fab_host_bar = g->di->host_bar;
        } catch (CommError& e) {
            set_err(GALA_E_NCCL, "%s", e.msg.c_str());
            throw GalaError{GALA_E_NCCL};
        }
        Comm& cm = *g->di->comm;
        g->di->v0 = v_begin;
        g->di->v1 = v_end;
        // every rank's owned range (ranges must tile [0, n) in rank order)
        const std::vector<int64_t> b0 = cm.allgather_host(v_begin, st), b1 = cm.allgather_host(v_end, st);
        g->dbounds0.assign(world + 1, 0);
        for (int r = 0; r < world; ++r) {
            if (b0[r] != (r ? b1[r - 1] : 0)) { set_err(GALA_E_INVALID, "owned ranges must tile [0, n) in rank order"); throw GalaError{GALA_E_INVALID}; }
            g->dbounds0[r] = b0[r];
        }
        g->dbounds0[world] = b1[world - 1];
        if (g->dbounds0[world] != n_global) { set_err(GALA_E_INVALID, "owned ranges do not cover n"); throw GalaError{GALA_E_INVALID}; }
        fabric_setup(g, *g->di, n_global);   // peer-memory region of the device-resident iteration (collective)
        const int64_t nnz = local_row_ptr[n_own];
        g->nnz0 = nnz;
        g->g0.n = n_global;
        g->g0.nnz = nnz;
        g->g0.rp = dalloc<int64_t>(n_global + 1, st);
        g->g0.col = dalloc<int32_t>(nnz, st);
        int64_t* lrp = dalloc<int64_t>(n_own + 1, st);
        CK(cudaMemcpyAsync(lrp, local_row_ptr, sizeof(int64_t) * (n_own + 1), cudaMemcpyHostToDevice, st));
        k_expand_rp<<<grid_for(n_global + 1, 256, g->num_sms * 8), 256, 0, st>>>(n_global, v_begin, v_end, lrp, g->g0.rp);
        CKL();
        dfree(lrp, st);
        if (nnz) CK(cudaMemcpyAsync(g->g0.col, col_idx, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, st));
        if (weights) {
            g->g0.w = dalloc<int64_t>(nnz, st);
            CK(cudaMemcpyAsync(g->g0.w, weights, sizeof(int64_t) * nnz, cudaMemcpyHostToDevice, st));
        }
        finish_graph(g);
        // unit-weight detection must agree on every rank
        const std::vector<int64_t> u = cm.allgather_host(g->g0.w ? 0 : 1, st);
        bool all_unit = true;
        for (int64_t x : u) all_unit = all_unit && x;
        if (!all_unit && !g->g0.w) {   // some rank has real weights: materialise ones here
            g->g0.w = dalloc<int64_t>(std::max<int64_t>(nnz, 1), st);
            k_fill_i64<<<grid_for(nnz, 256, g->num_sms * 8), 256, 0, st>>>(reinterpret_cast<long long*>(g->g0.w), nnz, 1);
            CKL();
        }
        // replicate d (owned slices), then W and the max weighted degree over all vertices
        std::vector<size_t> cb(world), db(world);
        for (int r = 0; r < world; ++r) {
            cb[r] = (size_t)(g->dbounds0[r + 1] - g->dbounds0[r]) * sizeof(int64_t);
            db[r] = (size_t)g->dbounds0[r] * sizeof(int64_t);
        }
        int64_t* dfull = dalloc<int64_t>(std::max<int64_t>(n_global, 1), st);
        cm.allgatherv(g->d0 + v_begin, dfull, cb, db, st);
        dfree(g->d0, st);
        g->d0 = dfull;
        const int big = g->num_sms * 8;
        i128* part = dalloc<i128>(big, st);
        ull* ticket = dalloc<ull>(1, st);
        i128* wsum = dalloc<i128>(1, st);
        ull* mx = dalloc<ull>(1, st);
        CK(cudaMemsetAsync(ticket, 0, sizeof(ull), st));
        CK(cudaMemsetAsync(mx, 0, sizeof(ull), st));
        k_sum_i128<<<grid_for(n_global, 256, big), 256, 0, st>>>(n_global, g->d0, part, ticket, wsum);
        CKL();
        k_max_i64<<<grid_for(n_global, 256, big), 256, 0, st>>>(n_global, g->d0, mx);
        CKL();
        i128 hW = 0;
        ull hm = 0;
        CK(cudaMemcpyAsync(&hW, wsum, sizeof(i128), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(&hm, mx, sizeof(ull), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        dfree(part, st); dfree(ticket, st); dfree(wsum, st); dfree(mx, st);
        if (hW >= ((i128)1 << 62)) { set_err(GALA_E_OVERFLOW, "total weight W >= 2^62"); throw GalaError{GALA_E_OVERFLOW}; }
        g->W = (int64_t)hW;
        g->maxw0 = (int64_t)hm;
        const std::vector<int64_t> rd = cm.allgather_host(g->rows_distinct0 ? 1 : 0, st);
        for (int64_t x : rd) g->rows_distinct0 = g->rows_distinct0 && x;
    } catch (...) {
        gala_graph_free(g);
        throw;
    }
    *out = g;
    API_END
}

}  // extern "C"
