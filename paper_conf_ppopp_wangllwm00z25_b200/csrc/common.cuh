// common.cuh — shared device types and helpers of the GALA sm_100a kernels.
//
// Exact integer arithmetic throughout (DESIGN.md "Readings" c1, c11, c16):
//   score(c) = qW * d_c(v) - p * Sig[c] * d(v)            (Eq. 2 x q W |E|)
//   stay     = qW * d'(v)  - p * (Sig[C[v]] - d(v)) * d(v) (v removed from its community)
// with gamma = p/q and W = 2|E|.  ST (score type) is int64 when
// max(p,q) * W * maxdeg < 2^62 on the level (chosen by the host), else __int128.
#pragma once

#include <cstdint>
#include <climits>
#include <cuda_runtime.h>

typedef __int128 i128;
typedef unsigned long long ull;

#define FULLMASK 0xffffffffu

// dispatch bins (a2): sub-warp groups of 4/8/16/32 lanes, warp hash (<=128, <=512), block hash,
// multi-block hub path (rows split into chunks)
enum { BIN_S4 = 0, BIN_S8 = 1, BIN_S16 = 2, BIN_S32 = 3, BIN_WARP = 4, BIN_WARP2 = 5, BIN_BLOCK = 6, BIN_HUB = 7,
       NBINS = 8 };

// Device-resident per-iteration counters (zeroed by k_iter_begin).
struct IterCounters {
    ull bin_count[NBINS];   // active vertices queued per bin
    ull bin_deg[NBINS];     // sum of row lengths of queued vertices (edges scanned)
    ull bin_k[NBINS];       // sum of distinct neighbour communities seen by decide
    ull n_active;
    ull n_pruned;
    ull n_moved;
    ull moved_deg;          // sum of row lengths of moved vertices
    ull cursor[NBINS];      // dynamic work cursors (block kernels)
    ull dp_mismatch;        // check mode: maintained d' != aggregated d'
    ull ticket;             // last-block-done ticket of k_reduce
    ull delta_used;         // 1 if the delta d' update ran this iteration
    ull cursor2;            // dynamic work cursor of the hub evaluation
    ull n_items;            // delta-update work items (one per light mover, one per chunk of a heavy one)
    ull n_fn;               // instrumented pruning: pruned vertices that would have moved (Eq. 3)
    ull n_fp;               // instrumented pruning: active vertices that stay
    ull cursor_hi;          // dynamic work cursor of the block bin's long-row class (k_decide_block CLS 2)
    ull n_items_hi;         // delta-update items of movers with rows > DLIGHT, stored from the END of the item arrays
    ull h0_acc, h1_acc;     // block-bin hash inserts landing in the shared H0 / the global H1 (§4.2 access rate)
    ull h0_keys, h1_keys;   // distinct communities held in H0 / H1 (§4.2 maintenance rate)
    ull n_dense;            // multi-GPU (fabric): senders whose label exchange went dense this iteration
    ull xbytes;             // multi-GPU (fabric): bytes this rank received in its inbox this iteration
};

// Pruning strategy of the active set (§3.2-3.3; DESIGN.md c20/c21):
//   0 none, 1 MG (Eq. 6/7), 2 SM (strict movement), 3 RM (relaxed movement), 4 MG+RM.
// The movement history of the previous iteration lives in per-vertex /
// per-community arrays holding the iteration id of the last event (-1 = never
// on this level), so nothing has to be cleared between iterations.
struct PruneState {
    int mode;
    int instr;          // 1: queue pruned vertices too, count n_fn / n_fp, apply only active moves
    int32_t* rmflag;    // RM: iteration in which some neighbour of v last moved
    int32_t* smflag;    // SM: iteration in which some neighbour community of v last changed
    int32_t* chg;       // SM: iteration in which community c last gained or lost a member
};

// Queue record of an active vertex, written by k_prune_bin (which already
// reads these fields) so the decide kernels start from one coalesced 48-byte
// load instead of a chain of dependent gathers.
struct __align__(16) QRec {
    int v;          // vertex
    int deg;        // row length
    long long beg;  // row_ptr[v]
    int cv;         // C[v]
    int szv;        // size[C[v]]
    long long dv;   // d(v)
    long long sigv; // Sigma_tot[C[v]]
    long long pad;
};

// Bin queues: bins 2r and 2r+1 share region r of `qstride` records, the even
// bin filling it upwards from the start and the odd one downwards from the end
// (their counts sum to at most the number of vertices), so NBINS/2 regions hold
// every queue.
struct QView {
    QRec* base;
    int dir;
    __host__ __device__ __forceinline__ QRec& operator[](long long i) const { return base[dir * i]; }
};
__host__ __device__ __forceinline__ QView qview(QRec* queues, long long qstride, int b) {
    QRec* r = queues + (long long)(b >> 1) * qstride;
    return (b & 1) ? QView{r + qstride - 1, -1} : QView{r, 1};
}

// Device-resident state carried across iterations of a level.
struct Carry {
    long long N_hi;         // current numerator N (int128 split)
    ull N_lo;
    long long N_prev_hi;    // numerator before this iteration
    ull N_prev_lo;
    long long minSig;       // min{Sig[c] : Sig[c] > 0}
    long long sumDC;        // sum_v (d'(v) + s(v))
    long long S2_hi;        // sum_c Sig[c]^2 (int128 split)
    ull S2_lo;
    int converged;
    int iter;               // iteration index within the level (also the d' stamp id)
    int more;               // loop condition written by k_record
    int log_base;           // log slot of iteration `log_base` is 0
    int ckey_valid;         // the per-entry community array matches C (set by full d' passes)
    int pad2;
    ull t_ns;               // %globaltimer at the end of the last reduction (level start / iteration end)
};

// One record per phase-1 iteration, written on the device by k_record.
struct IterLog {
    IterCounters ctr;
    long long N_hi;
    ull N_lo;
    int converged;
    int pad;
    ull t_ns;   // %globaltimer when the iteration's reduction finished (per-iteration device timing)
};

__device__ __forceinline__ ull globaltimer_ns() {
    ull t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ i128 mk128(long long hi, ull lo) {
    return (i128)(((unsigned __int128)(ull)hi << 64) | (unsigned __int128)lo);
}
__device__ __forceinline__ long long hi128(i128 x) { return (long long)(x >> 64); }
__device__ __forceinline__ ull lo128(i128 x) { return (ull)x; }

// warp shuffles for score types
__device__ __forceinline__ long long shfl_xor_st(long long x, int off) {
    return __shfl_xor_sync(FULLMASK, x, off);
}
__device__ __forceinline__ i128 shfl_xor_st(i128 x, int off) {
    long long h = __shfl_xor_sync(FULLMASK, (long long)(x >> 64), off);
    ull l = __shfl_xor_sync(FULLMASK, (ull)x, off);
    return mk128(h, l);
}
template <typename ST> __device__ __forceinline__ ST st_min();
template <> __device__ __forceinline__ long long st_min<long long>() { return LLONG_MIN; }
template <> __device__ __forceinline__ i128 st_min<i128>() { return mk128(LLONG_MIN, 0); }

// (score, community) ordering: higher score first, then lower community id.
template <typename ST>
__device__ __forceinline__ bool better(ST s1, int c1, ST s2, int c2) {
    return s1 > s2 || (s1 == s2 && c1 < c2);
}

// multiplicative hash of a community id into a power-of-two table
__device__ __forceinline__ unsigned hash_slot(int c, unsigned mask) {
    return ((unsigned)c * 2654435761u) & mask;
}
__device__ __forceinline__ unsigned hash_slot2(int c, unsigned mask) {
    return (((unsigned)c ^ 0x5bd1e995u) * 0x9E3779B1u >> 7) & mask;
}

// 16-byte volatile load of four consecutive table keys (generic address: shared or global)
__device__ __forceinline__ int4 ld_volatile_i4(const int* p) {
    int4 r;
    asm volatile("ld.volatile.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ int4 lds_volatile_i4(const int* p) {   // p points into shared memory
    int4 r;
    const unsigned a = (unsigned)__cvta_generic_to_shared(p);
    asm volatile("ld.volatile.shared.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(a));
    return r;
}
template <bool SH>
__device__ __forceinline__ int4 ld_bucket(const int* p) { return SH ? lds_volatile_i4(p) : ld_volatile_i4(p); }
// bit i set iff lane i of the 4-key bucket equals x
__device__ __forceinline__ unsigned match4(const int4& k, int x) {
    return (unsigned)(k.x == x) | ((unsigned)(k.y == x) << 1) | ((unsigned)(k.z == x) << 2) | ((unsigned)(k.w == x) << 3);
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// warp-aggregated append of a flagged lane's item to a queue; returns slot or -1
__device__ __forceinline__ long long warp_append(bool flag, ull* counter) {
    unsigned m = __ballot_sync(FULLMASK, flag);
    if (!m) return -1;
    int leader = __ffs(m) - 1;
    ull base = 0;
    if (lane_id() == leader) base = atomicAdd(counter, (ull)__popc(m));
    base = __shfl_sync(FULLMASK, base, leader);
    return flag ? (long long)(base + __popc(m & lanemask_lt())) : -1;
}

// Sum of `x` over the lanes of this lane's __match_any_sync group `peers`
// (the match_any + reduce pattern of Alg. 2).  Each lane adds its
// value into the group leader's slot of a per-warp shared scratch (32 slots).
// redux.sync is not used: with several groups per warp (different masks) it
// falls into a per-group serial path on sm_100.  32-bit adds are native
// shared atomics; the 64-bit variant (used only when sums can reach 2^32) is a
// CAS loop in hardware, hence the 32-bit aggregates wherever they suffice.
__device__ __forceinline__ unsigned group_sum(unsigned peers, unsigned x, unsigned* scratch) {
    const int lane = threadIdx.x & 31, leader = __ffs(peers) - 1;
    scratch[lane] = 0;
    __syncwarp();
    if (x) atomicAdd(&scratch[leader], x);
    __syncwarp();
    const unsigned r = scratch[leader];
    __syncwarp();
    return r;
}
__device__ __forceinline__ ull group_sum(unsigned peers, ull x, ull* scratch) {
    const int lane = threadIdx.x & 31, leader = __ffs(peers) - 1;
    scratch[lane] = 0;
    __syncwarp();
    if (x) atomicAdd(&scratch[leader], x);
    __syncwarp();
    const ull r = scratch[leader];
    __syncwarp();
    return r;
}

// warp-aggregated append of the lanes with `fresh` set (within group mask gmask)
// to list[*cnt ...]: one shared atomic per group instead of one per lane.  All
// 32 lanes must call it converged.
template <typename LT>
__device__ __forceinline__ void append_fresh(bool fresh, int slot, unsigned gmask, int* cnt, LT* list) {
    const int lane = threadIdx.x & 31;
    const unsigned fm = __ballot_sync(FULLMASK, fresh) & gmask;
    int base = 0;
    if (fresh && lane == __ffs(fm) - 1) base = atomicAdd(cnt, __popc(fm));
    base = __shfl_sync(FULLMASK, base, fm ? __ffs(fm) - 1 : lane);
    if (fresh) {
        unsigned lt;
        asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
        list[base + __popc(fm & lt)] = (LT)slot;
    }
}

__device__ __forceinline__ long long warp_sum_ll(long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(FULLMASK, x, o);
    return x;
}
