// k_phase2.cuh — device scan and phase-2 kernels: min-member relabel,
// label composition, and coarsening of communities into super vertices with
// per-community hash aggregation of super edges.  SURVEY.md §8(a) a8, a9.
#pragma once
#include "common.cuh"

// ---------------------------------------------------------------------------
// exclusive prefix sum of int64 (3 passes: tile sums, scan of sums, tile scan)
// out[i] = sum_{j<i} in[i]; out[n] = total.  in may alias out.
// ---------------------------------------------------------------------------
#define SCAN_BT 256
#define SCAN_IPT 8
#define SCAN_TILE (SCAN_BT * SCAN_IPT)

__device__ __forceinline__ long long block_excl_scan(long long x, long long* total) {
    __shared__ long long ws[SCAN_BT / 32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    long long inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        long long y = __shfl_up_sync(FULLMASK, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) ws[wib] = inc;
    __syncthreads();
    if (wib == 0) {
        long long t = lane < SCAN_BT / 32 ? ws[lane] : 0;
        long long ti = t;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            long long y = __shfl_up_sync(FULLMASK, ti, o);
            if (lane >= o) ti += y;
        }
        if (lane < SCAN_BT / 32) ws[lane] = ti - t;
        if (lane == SCAN_BT / 32 - 1) *total = ti;
    }
    __syncthreads();
    long long r = inc - x + ws[wib];
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(SCAN_BT) k_scan_tiles(const long long* __restrict__ in, long long n,
                                                        long long* __restrict__ sums) {
    __shared__ long long tot;
    long long base = (long long)blockIdx.x * SCAN_TILE + (long long)threadIdx.x * SCAN_IPT;
    long long x = 0;
#pragma unroll
    for (int i = 0; i < SCAN_IPT; ++i)
        if (base + i < n) x += in[base + i];
    block_excl_scan(x, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// single block: exclusive scan of the tile sums in place (chunks of SCAN_BT)
__global__ void __launch_bounds__(SCAN_BT) k_scan_sums(long long* __restrict__ sums, long long nt) {
    __shared__ long long tot;
    long long carry = 0;
    for (long long b = 0; b < nt; b += SCAN_BT) {
        long long i = b + threadIdx.x;
        long long x = i < nt ? sums[i] : 0;
        long long e = block_excl_scan(x, &tot);
        if (i < nt) sums[i] = carry + e;
        carry += tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) sums[nt] = carry;
}

__global__ void __launch_bounds__(SCAN_BT) k_scan_apply(const long long* in, long long n,
                                                        const long long* __restrict__ sums, long long* out,
                                                        long long nt) {
    __shared__ long long tot;
    long long base = (long long)blockIdx.x * SCAN_TILE + (long long)threadIdx.x * SCAN_IPT;
    long long v[SCAN_IPT];
    long long x = 0;
#pragma unroll
    for (int i = 0; i < SCAN_IPT; ++i) {
        v[i] = (base + i < n) ? in[base + i] : 0;
        x += v[i];
    }
    long long e = block_excl_scan(x, &tot) + sums[blockIdx.x];
#pragma unroll
    for (int i = 0; i < SCAN_IPT; ++i) {
        if (base + i < n) out[base + i] = e;
        e += v[i];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) out[n] = sums[nt];
}

// ---------------------------------------------------------------------------
// a8: relabel in min-member order (reading c9) and compose the global map
// ---------------------------------------------------------------------------
__global__ void k_fill_i32(int32_t* p, long long n, int32_t val) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        p[i] = val;
}
__global__ void k_fill_i64(long long* p, long long n, long long val) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        p[i] = val;
}

__global__ void k_minmember(int n, const int32_t* __restrict__ C, int32_t* __restrict__ minmem) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
        atomicMin(&minmem[C[v]], (int32_t)v);
}

// flag[v] = 1 iff v is the smallest member of its community
__global__ void k_minflag(int n, const int32_t* __restrict__ C, const int32_t* __restrict__ minmem,
                          long long* __restrict__ flag) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
        flag[v] = (minmem[C[v]] == v) ? 1 : 0;
}

// newid[v] = rank of v's community = pos[minmem[C[v]]]
__global__ void k_newid(int n, const int32_t* __restrict__ C, const int32_t* __restrict__ minmem,
                        const long long* __restrict__ pos, int32_t* __restrict__ newid) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
        newid[v] = (int32_t)pos[minmem[C[v]]];
}

__global__ void k_compose(long long n0, const int32_t* __restrict__ newid, int32_t* __restrict__ lab) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n0; v += (long long)gridDim.x * blockDim.x)
        lab[v] = newid[lab[v]];
}

// ---------------------------------------------------------------------------
// a9: coarsen.  Super vertex c' = newid of a community; super edge (c', x')
// weight = sum of w(v,u) over entries with newid[v] = c', newid[u] = x'.
// The diagonal (internal weight D_C, reading c10) is one entry.
// ---------------------------------------------------------------------------
// Coarsening runs per community c' = newid of a community:
//   1. k_comm_stats  : row entries per community -> eoff (exclusive scan)
//   2. k_gather_rows : every row's coarse keys newid[u] (and weights) are copied
//                      into its community's contiguous segment [eoff[c'], eoff[c'+1])
//   3. aggregation of each segment into a hash table keyed by coarse neighbour,
//      by the cheapest path that fits:
//        k_agg_warp  (table <= 256 slots, one warp per community),
//        k_agg_block (table <= smem capacity, one block per community),
//        k_agg_big_* (larger: global table shared by BPC blocks);
//      segments are read coalesced, 4 entries per lane in flight, equal keys of
//      every 32-entry chunk combined with __match_any_sync before inserting;
//      distinct entries are written back to the segment start, their count to
//      dn[c'], the diagonal weight to snew[c'].
//   4. k_compact     : segments -> coarse CSR rows (rp_new = scan of dn).
// Tables live in shared memory on the common paths (P:304-316's point about
// keeping hot state on chip applies to phase 2 as well).
__global__ void k_comm_stats(int n, const int64_t* __restrict__ rp, const int32_t* __restrict__ newid,
                             long long* __restrict__ ent) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
        long long dg = rp[v + 1] - rp[v];
        if (dg) atomicAdd(reinterpret_cast<ull*>(&ent[newid[v]]), (ull)dg);
    }
}

// segment position of every row: eoff[c'] + its offset among c's rows
__global__ void k_vpos(int n, const int64_t* __restrict__ rp, const int32_t* __restrict__ newid,
                       const long long* __restrict__ eoff, long long* __restrict__ ecur, long long* __restrict__ vpos) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
        const long long dg = rp[v + 1] - rp[v];
        const int c = newid[v];
        vpos[v] = dg ? eoff[c] + (long long)atomicAdd(reinterpret_cast<ull*>(&ecur[c]), (ull)dg) : 0;
    }
}

// Few communities (k <= AGG_HIST_K): the per-community sums above hit the same few counters
// from every thread (thousands of same-address atomics each).  These variants first count in a
// block-local shared histogram over a contiguous tile of AGG_HIST_T vertices, then add each
// nonzero bin once per block; k_vpos_hist also hands every vertex its offset inside the block's
// share of its community segment.
#define AGG_HIST_K 4096
#define AGG_HIST_T 2048
__global__ void __launch_bounds__(256) k_comm_stats_hist(int n, long long k, const int64_t* __restrict__ rp,
                                                         const int32_t* __restrict__ newid, long long* __restrict__ ent) {
    extern __shared__ unsigned hist[];
    for (long long c = threadIdx.x; c < k; c += 256) hist[c] = 0;
    __syncthreads();
    const long long v0 = (long long)blockIdx.x * AGG_HIST_T;
    for (long long v = v0 + threadIdx.x; v < min((long long)n, v0 + AGG_HIST_T); v += 256) {
        const long long dg = rp[v + 1] - rp[v];
        if (dg) atomicAdd(&hist[newid[v]], (unsigned)dg);
    }
    __syncthreads();
    for (long long c = threadIdx.x; c < k; c += 256)
        if (hist[c]) atomicAdd(reinterpret_cast<ull*>(&ent[c]), (ull)hist[c]);
}
__global__ void __launch_bounds__(256) k_vpos_hist(int n, long long k, const int64_t* __restrict__ rp,
                                                   const int32_t* __restrict__ newid, const long long* __restrict__ eoff,
                                                   long long* __restrict__ ecur, long long* __restrict__ vpos) {
    extern __shared__ unsigned char hraw[];
    unsigned* hist = reinterpret_cast<unsigned*>(hraw);
    long long* base = reinterpret_cast<long long*>(hraw + ((k * sizeof(unsigned) + 15) & ~(long long)15));
    constexpr int PER = AGG_HIST_T / 256;
    for (long long c = threadIdx.x; c < k; c += 256) hist[c] = 0;
    __syncthreads();
    const long long v0 = (long long)blockIdx.x * AGG_HIST_T;
    unsigned loc[PER];
    int cc[PER];
    long long dgs[PER];
#pragma unroll
    for (int t = 0; t < PER; ++t) {
        const long long v = v0 + threadIdx.x + 256 * t;
        dgs[t] = v < n ? rp[v + 1] - rp[v] : 0;
        cc[t] = v < n ? newid[v] : 0;
        loc[t] = dgs[t] ? atomicAdd(&hist[cc[t]], (unsigned)dgs[t]) : 0;
    }
    __syncthreads();
    for (long long c = threadIdx.x; c < k; c += 256)
        base[c] = hist[c] ? (long long)atomicAdd(reinterpret_cast<ull*>(&ecur[c]), (ull)hist[c]) : 0;
    __syncthreads();
#pragma unroll
    for (int t = 0; t < PER; ++t) {
        const long long v = v0 + threadIdx.x + 256 * t;
        if (v < n) vpos[v] = dgs[t] ? eoff[cc[t]] + base[cc[t]] + loc[t] : 0;
    }
}

// per-entry weights of the community-major segments: 32-bit when every aggregated weight fits
// (W < 2^32, the common case: the level-0 graph of every config), else 64-bit
struct TVal {
    void* p;
    int w32;
    __device__ __forceinline__ long long get(long long j) const {
        return w32 ? (long long)static_cast<const unsigned*>(p)[j] : static_cast<const long long*>(p)[j];
    }
    __device__ __forceinline__ void set(long long j, long long v) const {
        if (w32) static_cast<unsigned*>(p)[j] = (unsigned)v;
        else static_cast<long long*>(p)[j] = v;
    }
};

// edge-parallel: entry e of row r goes to vpos[r] + (e - rp[r]) with key newid[col[e]];
// 4 entries per lane in flight, coalesced row/col streams
template <bool UNIT>
__global__ void __launch_bounds__(256) k_gather_flat(long long nnz, const int32_t* __restrict__ row,
                                                     const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                     const int64_t* __restrict__ w, const int32_t* __restrict__ newid,
                                                     const long long* __restrict__ vpos, int* __restrict__ tkey,
                                                     TVal tval) {
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long base = (((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 128; base < nnz;
         base += nw * 128) {
        int r[4], u[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            long long e = base + lane + 32 * t;
            r[t] = e < nnz ? row[e] : 0;
            u[t] = e < nnz ? col[e] : 0;
        }
        int kk[4];
        long long dst[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            long long e = base + lane + 32 * t;
            kk[t] = e < nnz ? newid[u[t]] : 0;
            dst[t] = e < nnz ? vpos[r[t]] + (e - rp[r[t]]) : 0;
        }
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            long long e = base + lane + 32 * t;
            if (e < nnz) {
                tkey[dst[t]] = kk[t];
                if (!UNIT) tval.set(dst[t], w[e]);
            }
        }
    }
}

// ---------------------------------------------------------------------------
// a9, few communities (k <= AGG_DENSE_K): the coarse graph has at most k^2 entries, so it is
// accumulated straight into a dense k x k matrix M (L2-resident: 1202^2 x 4 B = 5.8 MB for the
// Orkut-shaped level 0) -- no community-major segments, no hash tables.  Edge-parallel over the
// CSR (4 entries per lane in flight); the entries of a 32-entry chunk with the same (c1, c2) are
// combined with __match_any_sync first, so the diagonal (most entries of a good partition) sees
// one atomic per chunk.  M[c][c] is D_C(c) (every entry inside c, reading c10).  Rows are then
// counted, scanned and emitted in ascending column order.
// ---------------------------------------------------------------------------
#define AGG_DENSE_K 4096
template <bool UNIT, typename V>
__global__ void __launch_bounds__(256) k_agg_dense_accum(long long nnz, const int32_t* __restrict__ row,
                                                         const int32_t* __restrict__ col, const int64_t* __restrict__ w,
                                                         const int32_t* __restrict__ newid,
                                                         const int32_t* __restrict__ keymap, long long k,
                                                         V* __restrict__ M) {
    __shared__ V s_scr[8][32];   // per-warp group sums (weighted levels)
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long base = (((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 128; base < nnz;
         base += nw * 128) {
        int r[4], u[4];
        V wt[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const long long e = base + lane + 32 * t;
            r[t] = e < nnz ? row[e] : -1;
            u[t] = e < nnz ? col[e] : 0;
            wt[t] = (e < nnz && !UNIT) ? (V)w[e] : (V)1;
        }
        long long key[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) key[t] = r[t] >= 0 ? (long long)newid[r[t]] * k + keymap[u[t]] : -1 - lane;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const unsigned peers = __match_any_sync(FULLMASK, key[t]);
            const V sum = UNIT ? (V)__popc(peers) : group_sum(peers, r[t] >= 0 ? wt[t] : (V)0, s_scr[threadIdx.x >> 5]);
            if (r[t] >= 0 && lane == __ffs(peers) - 1) atomicAdd(&M[key[t]], sum);
        }
    }
}

// warp per coarse row: distinct entries -> dn[c], diagonal -> snew[c]
template <typename V>
__global__ void k_agg_dense_count(long long k, const V* __restrict__ M, long long* __restrict__ dn,
                                  int64_t* __restrict__ snew) {
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long c = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < k; c += nw) {
        const V* rowp = M + c * k;
        long long cnt = 0;
        for (long long j = lane; j < k; j += 32) cnt += rowp[j] != 0;
        cnt = warp_sum_ll(cnt);
        if (lane == 0) { dn[c] = cnt; snew[c] = (int64_t)rowp[c]; }
    }
}

// warp per coarse row: nonzeros in ascending column order -> CSR (col, w, row); M cleared
template <typename V>
__global__ void k_agg_dense_emit(long long k, V* __restrict__ M, const long long* __restrict__ rp,
                                 int32_t* __restrict__ ocol, int64_t* __restrict__ ow, int32_t* __restrict__ orow) {
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long c = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < k; c += nw) {
        V* rowp = M + c * k;
        long long o = rp[c];
        for (long long j0 = 0; j0 < k; j0 += 32) {
            const long long j = j0 + lane;
            const V x = j < k ? rowp[j] : (V)0;
            const unsigned nz = __ballot_sync(FULLMASK, x != 0);
            if (x != 0) {
                const long long at = o + __popc(nz & lanemask_lt());
                ocol[at] = (int32_t)j;
                ow[at] = (int64_t)x;
                orow[at] = (int32_t)c;
                rowp[j] = 0;
            }
            o += __popc(nz);
        }
    }
}

// row id of every CSR entry (warp per row)
__global__ void k_fill_rows(int n, const int64_t* __restrict__ rp, int32_t* __restrict__ row) {
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long v = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < n; v += nw)
        for (int64_t j = rp[v] + lane; j < rp[v + 1]; j += 32) row[j] = (int32_t)v;
}

// table capacity a community needs: nextpow2(2 * min(entries, k)) (0 if no entries)
__device__ __forceinline__ long long agg_cap(long long ent, long long k) {
    if (ent == 0) return 0;
    const long long m = ent < k ? ent : k;
    return 1LL << (64 - __clzll(2 * m - 1));
}

struct AggArgs {
    long long k;
    const long long* ent;
    const long long* eoff;     // segment offsets (exclusive scan of ent)
    int* tkey;                 // segments: coarse keys in, distinct keys out
    TVal tval;                 // weights in (weighted levels), aggregated weights out
    long long* dn;             // distinct entries per community
    int64_t* snew;             // diagonal weight per community
};

// open-addressing insert / accumulate (slot-wise linear probe; tables are never full: cap >= 2 x
// distinct keys).  Returns the slot, *fresh when this lane created the key; the caller appends
// the warp's fresh slots to the distinct list with ONE counter atomic (append_fresh) -- a per-key
// append serialised the 32 lanes of a chunk on one shared counter whenever most keys were new.
template <typename VT>
__device__ __forceinline__ int agg_insert_nl(int key, VT wt, int* keys, VT* vals, unsigned mask, bool* fresh) {
    unsigned h = hash_slot(key, mask);
    for (;;) {
        int k0 = *(volatile int*)&keys[h];
        if (k0 == key) { atomicAdd(&vals[h], wt); *fresh = false; return (int)h; }
        if (k0 == -1) {
            int old = atomicCAS(&keys[h], -1, key);
            if (old == -1 || old == key) { atomicAdd(&vals[h], wt); *fresh = old == -1; return (int)h; }
        }
        h = (h + 1) & mask;
    }
}

// Global-table form for a whole warp (all 32 lanes call it, converged; `on` marks lanes with a key):
// insert / accumulate without touching the list, then append the warp's fresh slots with ONE
// returning atomic on the community's list counter (every block working on a community hits that
// counter; one atomic per fresh key serialised them -- the friendster_q level-0 coarsening).
template <typename GV>
__device__ __forceinline__ void agg_insert_warp(bool on, int key, GV wt, int* keys, GV* vals, unsigned mask,
                                                int* list, int* cnt) {
    bool fresh = false;
    unsigned h = 0;
    if (on) {
        h = hash_slot(key, mask);
        for (;;) {
            const int k0 = *(volatile int*)&keys[h];
            if (k0 == key) { atomicAdd(&vals[h], wt); break; }
            if (k0 == -1) {
                const int old = atomicCAS(&keys[h], -1, key);
                if (old == -1 || old == key) { fresh = old == -1; atomicAdd(&vals[h], wt); break; }
            }
            h = (h + 1) & mask;
        }
    }
    const unsigned fm = __ballot_sync(FULLMASK, fresh);
    if (!fm) return;
    const int lane = threadIdx.x & 31, lead = __ffs(fm) - 1;
    int base = 0;
    if (lane == lead) base = atomicAdd(cnt, __popc(fm));
    base = __shfl_sync(FULLMASK, base, lead);
    if (fresh) list[base + __popc(fm & ((1u << lane) - 1u))] = (int)h;
}

// `nt` threads (tid = this thread's index among them, whole warps) stream
// segment entries [s0, s1) with 4 entries per lane in flight; equal keys of
// every 32-entry chunk are combined before inserting.
// TV: table value type; SV: per-chunk group-sum type (32-bit whenever W < 2^32, so
// the shared-memory adds are native)
template <bool UNIT, typename TV, typename SV>
__device__ __forceinline__ void agg_segment(const AggArgs& a, long long s0, long long s1, int tid, int nt, int* keys,
                                            TV* vals, unsigned mask, int* list, int* cnt, SV* scratch) {
    const int lane = tid & 31;
    for (long long r0 = s0 + (tid & ~31) * 4; r0 < s1; r0 += (long long)nt * 4) {   // warp-uniform
        int kk[4];
        SV ww[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            long long j = r0 + lane + 32 * t;
            kk[t] = j < s1 ? a.tkey[j] : -1;
            ww[t] = (j < s1 && !UNIT) ? (SV)a.tval.get(j) : (SV)1;
        }
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            if (r0 + 32 * t >= s1) break;
            const unsigned peers = __match_any_sync(FULLMASK, kk[t] >= 0 ? kk[t] : -1 - lane);
            const SV sum = UNIT ? (SV)__popc(peers) : group_sum(peers, kk[t] >= 0 ? ww[t] : (SV)0, scratch);
            bool fresh = false;
            int slot = -1;
            if (kk[t] >= 0 && lane == __ffs(peers) - 1) slot = agg_insert_nl<TV>(kk[t], (TV)sum, keys, vals, mask, &fresh);
            append_fresh<int>(fresh, slot, FULLMASK, cnt, list);   // one list-counter atomic per warp
        }
    }
}

// write the distinct entries of community c to the start of its segment
template <typename VT>
__device__ __forceinline__ void agg_emit(const AggArgs& a, long long c, int m, const int* list, int* keys, VT* vals,
                                         int tid, int nt) {
    const long long o = a.eoff[c];
    for (int t = tid; t < m; t += nt) {
        int slot = list[t];
        int key = keys[slot];
        int64_t val = (int64_t)vals[slot];
        keys[slot] = -1;
        vals[slot] = 0;
        a.tkey[o + t] = key;
        a.tval.set(o + t, val);
        if (key == (int)c) a.snew[c] = val;
    }
}

#define AGG_WSLOTS 256
template <bool UNIT, typename V>
__global__ void __launch_bounds__(256) k_agg_warp(AggArgs a, const int32_t* __restrict__ wl,
                                                  const int* __restrict__ nwl) {
    __shared__ __align__(16) int s_key[8][AGG_WSLOTS];
    __shared__ V s_val[8][AGG_WSLOTS];
    __shared__ int s_list[8][AGG_WSLOTS / 2];
    __shared__ int s_cnt[8];
    __shared__ V s_scr[8][32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    int* keys = s_key[wib];
    V* vals = s_val[wib];
    int* list = s_list[wib];
    for (int j = lane; j < AGG_WSLOTS; j += 32) { keys[j] = -1; vals[j] = 0; }
    if (lane == 0) s_cnt[wib] = 0;
    __syncwarp();
    const long long nw = (long long)gridDim.x * 8;
    const long long cnt = *nwl;
    for (long long i = (long long)blockIdx.x * 8 + wib; i < cnt; i += nw) {
        const long long c = wl[i];
        const long long s0 = a.eoff[c], s1 = a.eoff[c + 1];
        if (s1 - s0 <= 32) {   // one lane per entry: __match_any_sync alone finds the distinct keys
            const int j = lane;
            const bool on = j < s1 - s0;
            const int key = on ? a.tkey[s0 + j] : -1 - lane;
            const V wt = (on && !UNIT) ? (V)a.tval.get(s0 + j) : (V)(on ? 1 : 0);
            const unsigned peers = __match_any_sync(FULLMASK, key);
            const V sum = UNIT ? (V)__popc(peers) : group_sum(peers, wt, s_scr[wib]);
            const bool lead = on && lane == __ffs(peers) - 1;
            const unsigned lm = __ballot_sync(FULLMASK, lead);
            if (lead) {   // distinct entries to the start of the segment (lead lanes ascend, never overtake)
                const int t = __popc(lm & lanemask_lt());
                a.tkey[s0 + t] = key;
                a.tval.set(s0 + t, (int64_t)sum);
                if (key == (int)c) a.snew[c] = (int64_t)sum;
            }
            if (lane == 0) a.dn[c] = __popc(lm);
            continue;
        }
        const long long cap = agg_cap(a.ent[c], a.k);
        agg_segment<UNIT, V, V>(a, s0, s1, lane, 32, keys, vals, (unsigned)cap - 1, list,
                                &s_cnt[wib], s_scr[wib]);
        __syncwarp();
        int m = s_cnt[wib];
        agg_emit<V>(a, c, m, list, keys, vals, lane, 32);
        __syncwarp();
        if (lane == 0) { a.dn[c] = m; s_cnt[wib] = 0; }
        __syncwarp();
    }
}

template <int BT, bool UNIT, typename V>
__global__ void __launch_bounds__(BT) k_agg_block(AggArgs a, int scap, const int32_t* __restrict__ bl,
                                                  const int* __restrict__ nbl) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    V* vals = reinterpret_cast<V*>(smem_raw);
    int* keys = reinterpret_cast<int*>(smem_raw + (size_t)scap * sizeof(V));
    int* list = keys + scap;
    __shared__ int s_cnt;
    __shared__ V s_scr[BT / 32][32];
    const int wib = threadIdx.x >> 5;
    for (int j = threadIdx.x; j < scap; j += BT) { keys[j] = -1; vals[j] = 0; }
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    const long long cnt = *nbl;
    for (long long i = blockIdx.x; i < cnt; i += gridDim.x) {
        const long long c = bl[i];
        const long long cap = agg_cap(a.ent[c], a.k);
        agg_segment<UNIT, V, V>(a, a.eoff[c], a.eoff[c + 1], threadIdx.x, BT, keys, vals, (unsigned)cap - 1, list,
                                &s_cnt, s_scr[wib]);
        __syncthreads();
        int m = s_cnt;
        agg_emit<V>(a, c, m, list, keys, vals, threadIdx.x, BT);
        __syncthreads();
        if (threadIdx.x == 0) { a.dn[c] = m; s_cnt = 0; }
        __syncthreads();
    }
}

// Class D: communities whose table bound (2 min(entries, k)) exceeds the shared arena but whose
// segment is short enough for one block (entries <= agg_big_ent): the hierarchical table of §4.2
// -- the block's shared H0 (scap slots, probed over a window of AGG_HWIN slots once
// the bound exceeds it) spills to the block's own global H1 (linear probing, sized for the
// longest class-D segment), both with distinct lists.  The bound is pessimistic (the Friendster-
// shaped level 0 averages ~5k distinct keys in ~15k entries), so almost every key stays in H0
// and the chunked global path (every key a global atomic) is left to the truly big communities.
#define AGG_HWIN 32
template <bool UNIT, typename V>
__global__ void __launch_bounds__(512) k_agg_block_h(AggArgs a, int scap, const int32_t* __restrict__ bl,
                                                     const int* __restrict__ nbl, int* __restrict__ gkeys_all,
                                                     ull* __restrict__ gvals_all, int* __restrict__ glist_all,
                                                     long long gcap) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    V* vals = reinterpret_cast<V*>(smem_raw);
    int* keys = reinterpret_cast<int*>(smem_raw + (size_t)scap * sizeof(V));
    int* list = keys + scap;
    __shared__ int s_cnt, s_gcnt;
    __shared__ V s_scr[16][32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    int* gkeys = gkeys_all + (long long)blockIdx.x * gcap;
    ull* gvals = gvals_all + (long long)blockIdx.x * gcap;
    int* glist = glist_all + (long long)blockIdx.x * gcap;
    const unsigned smask = (unsigned)scap - 1, gmask = (unsigned)gcap - 1;
    for (int j = threadIdx.x; j < scap; j += 512) { keys[j] = -1; vals[j] = 0; }
    if (threadIdx.x == 0) { s_cnt = 0; s_gcnt = 0; }
    __syncthreads();
    const long long cnt = *nbl;
    for (long long i = blockIdx.x; i < cnt; i += gridDim.x) {
        const long long c = bl[i];
        const long long s0 = a.eoff[c], s1 = a.eoff[c + 1];
        for (long long r0 = s0 + (threadIdx.x & ~31) * 4; r0 < s1; r0 += 512LL * 4) {   // warp-uniform
            int kk[4];
            V ww[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const long long j = r0 + lane + 32 * t;
                kk[t] = j < s1 ? a.tkey[j] : -1;
                ww[t] = (j < s1 && !UNIT) ? (V)a.tval.get(j) : (V)1;
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (r0 + 32 * t >= s1) break;
                const unsigned peers = __match_any_sync(FULLMASK, kk[t] >= 0 ? kk[t] : -1 - lane);
                const V sum = UNIT ? (V)__popc(peers) : group_sum(peers, kk[t] >= 0 ? ww[t] : (V)0, s_scr[wib]);
                bool gfresh = false, sfresh = false;
                unsigned gh = 0, sh = 0;
                if (kk[t] >= 0 && lane == __ffs(peers) - 1) {
                    // H0: window of AGG_HWIN slots
                    unsigned h = hash_slot(kk[t], smask);
                    bool done = false;
                    for (int p = 0; p < AGG_HWIN && !done; ++p, h = (h + 1) & smask) {
                        const int k0 = keys[h];
                        if (k0 == kk[t]) { atomicAdd(&vals[h], sum); done = true; }
                        else if (k0 == -1) {
                            const int old = atomicCAS(&keys[h], -1, kk[t]);
                            if (old == -1) { atomicAdd(&vals[h], sum); sfresh = true; sh = h; done = true; }
                            else if (old == kk[t]) { atomicAdd(&vals[h], sum); done = true; }
                        }
                    }
                    if (!done) {   // H1
                        gh = hash_slot(kk[t], gmask);
                        for (;;) {
                            const int k0 = *(volatile int*)&gkeys[gh];
                            if (k0 == kk[t]) { atomicAdd(&gvals[gh], (ull)sum); break; }
                            if (k0 == -1) {
                                const int old = atomicCAS(&gkeys[gh], -1, kk[t]);
                                if (old == -1 || old == kk[t]) { gfresh = old == -1; atomicAdd(&gvals[gh], (ull)sum); break; }
                            }
                            gh = (gh + 1) & gmask;
                        }
                    }
                }
                append_fresh<int>(sfresh, (int)sh, FULLMASK, &s_cnt, list);   // one counter atomic per warp
                const unsigned fm = __ballot_sync(FULLMASK, gfresh);
                if (fm) {
                    const int lead = __ffs(fm) - 1;
                    int base = 0;
                    if (lane == lead) base = atomicAdd(&s_gcnt, __popc(fm));
                    base = __shfl_sync(FULLMASK, base, lead);
                    if (gfresh) glist[base + __popc(fm & lanemask_lt())] = (int)gh;
                }
            }
        }
        __syncthreads();
        const int m0 = s_cnt, m1 = s_gcnt;
        // distinct entries to the start of the segment (m0 + m1 <= entries), tables cleared
        for (int t = threadIdx.x; t < m0 + m1; t += 512) {
            int key;
            int64_t val;
            if (t < m0) {
                const int slot = list[t];
                key = keys[slot];
                val = (int64_t)vals[slot];
                keys[slot] = -1;
                vals[slot] = 0;
            } else {
                const int slot = glist[t - m0];
                key = gkeys[slot];
                val = (int64_t)gvals[slot];
                gkeys[slot] = -1;
                gvals[slot] = 0;
            }
            a.tkey[s0 + t] = key;
            a.tval.set(s0 + t, val);
            if (key == (int)c) a.snew[c] = val;
        }
        __syncthreads();
        if (threadIdx.x == 0) { a.dn[c] = m0 + m1; s_cnt = 0; s_gcnt = 0; }
        __syncthreads();
    }
}

// big communities: BPC blocks per community stream chunks of its segment into its global table
template <bool UNIT, typename V>
__global__ void __launch_bounds__(256) k_agg_big_insert(AggArgs a, const int32_t* __restrict__ bigc, int nbig,
                                                        const long long* __restrict__ goff, int* __restrict__ gkeys,
                                                        ull* __restrict__ gvals, int* __restrict__ glist,
                                                        int* __restrict__ gcnt, int bpc) {
    __shared__ V s_scr[8][32];
    const int wib = threadIdx.x >> 5;
    for (long long b = blockIdx.x; b < (long long)nbig * bpc; b += gridDim.x) {
        const int bi = (int)(b / bpc), part = (int)(b % bpc);
        const long long c = bigc[bi];
        const long long off = goff[bi];
        const unsigned mask = (unsigned)(goff[bi + 1] - off) - 1u;
        const long long s0 = a.eoff[c], len = a.eoff[c + 1] - s0;
        const long long lo = s0 + len * part / bpc, hi = s0 + len * (part + 1) / bpc;
        agg_segment<UNIT, ull, V>(a, lo, hi, threadIdx.x, 256, gkeys + off, gvals + off, mask, glist + off / 2,
                                  &gcnt[bi], s_scr[wib]);
    }
}

__global__ void __launch_bounds__(256) k_agg_big_emit(AggArgs a, const int32_t* __restrict__ bigc, int nbig,
                                                      const long long* __restrict__ goff, int* __restrict__ gkeys,
                                                      ull* __restrict__ gvals, const int* __restrict__ glist,
                                                      const int* __restrict__ gcnt, int bpc) {
    for (long long b = blockIdx.x; b < (long long)nbig * bpc; b += gridDim.x) {
        const int bi = (int)(b / bpc), part = (int)(b % bpc);
        const long long c = bigc[bi];
        const long long off = goff[bi];
        const int m = gcnt[bi];
        const int lo = (int)((long long)m * part / bpc), hi = (int)((long long)m * (part + 1) / bpc);
        const long long o = a.eoff[c];
        const int* list = glist + off / 2;
        for (int t = lo + threadIdx.x; t < hi; t += 256) {
            const int slot = list[t];
            const int key = gkeys[off + slot];
            const int64_t val = (int64_t)gvals[off + slot];
            a.tkey[o + t] = key;
            a.tval.set(o + t, val);
            if (key == (int)c) a.snew[c] = val;
        }
        if (part == 0 && threadIdx.x == 0) a.dn[c] = m;
    }
}

// Sort every community into the path that fits its table: warp (<= AGG_WSLOTS
// slots), block (<= scap), big (global table); communities without entries get
// dn = 0 here.  Lists are filled with warp-aggregated appends.
__device__ __forceinline__ void list_append(bool on, int32_t val, int32_t* list, int* cnt) {
    const unsigned m = __ballot_sync(FULLMASK, on);
    if (!m) return;
    const int lane = lane_id(), lead = __ffs(m) - 1;
    int base = 0;
    if (lane == lead) base = atomicAdd(cnt, __popc(m));
    base = __shfl_sync(FULLMASK, base, lead);
    if (on) list[base + __popc(m & lanemask_lt())] = val;
}

// block-path size classes (table slots): <= AGG_BA (BT 128), <= AGG_BB (BT 256), <= scap (BT 512)
#define AGG_BA 1024
#define AGG_BB 4096
__global__ void k_agg_classify(long long k, const long long* __restrict__ ent, int scap, long long* __restrict__ dn,
                               int32_t* __restrict__ wl, int* __restrict__ nwl, int32_t* __restrict__ bl,
                               int* __restrict__ nbl, int32_t* __restrict__ bigc, long long* __restrict__ bigcap,
                               int* __restrict__ nbig, long long kcap, long long big_ent, long long spill_ent) {
    // bl holds three lists of capacity kcap each (classes A, B, C), nbl their three counts;
    // communities with more than big_ent entries take the chunked big path even when their
    // table fits in shared memory (one block per community would serialise them)
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long c0 = (long long)blockIdx.x * blockDim.x; c0 < k; c0 += stride) {   // warp-uniform trips
        const long long c = c0 + threadIdx.x;
        const long long e = c < k ? ent[c] : 0;
        const long long cap = c < k ? agg_cap(e, k) : -1;
        if (cap == 0) dn[c] = 0;
        // class D (spilling block path, bl + 3 kcap): table beyond the arena, segment short enough
        const bool spill = cap > scap && e <= spill_ent;
        list_append(spill, (int32_t)c, bl + 3 * kcap, nbl + 3);
        const bool isbig = !spill && (cap > scap || e > big_ent);
        list_append(!isbig && cap > 0 && cap <= AGG_WSLOTS, (int32_t)c, wl, nwl);
        list_append(!isbig && cap > AGG_WSLOTS && cap <= AGG_BA && cap <= scap, (int32_t)c, bl, nbl);
        list_append(!isbig && cap > AGG_BA && cap <= AGG_BB && cap <= scap, (int32_t)c, bl + kcap, nbl + 1);
        list_append(!isbig && cap > AGG_BB && cap <= scap, (int32_t)c, bl + 2 * kcap, nbl + 2);
        const unsigned m = __ballot_sync(FULLMASK, isbig);
        if (m) {
            const int lane = lane_id(), lead = __ffs(m) - 1;
            int base = 0;
            if (lane == lead) base = atomicAdd(nbig, __popc(m));
            base = __shfl_sync(FULLMASK, base, lead);
            if (isbig) {
                const int i = base + __popc(m & lanemask_lt());
                bigc[i] = (int32_t)c;
                bigcap[i] = cap;
            }
        }
    }
}

// largest c in [lo, hi] with off[c] <= t
__device__ __forceinline__ long long seg_search(const long long* __restrict__ off, long long lo, long long hi,
                                                long long t) {
    while (lo < hi) {
        long long mid = (lo + hi + 1) >> 1;
        if (off[mid] <= t) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// Big communities (table larger than the block path's smem table): their
// segments are cut into AGG_CH-entry chunks; chunk t of all big communities
// (prefix choff; AGG_CH by default, option agg_chunk) is taken by any block of the machine, pre-combined in a
// block-local smem table, and only its distinct (key, sum) pairs are inserted
// into the community's global table (the global level of the hierarchy, as in
// the phase-1 hub path).  A giant community therefore spreads over every SM
// and its hot keys (the diagonal above all) see one global atomic per chunk.
#define AGG_CH 4096
#define AGG_CH_SLOTS (2 * AGG_CH)
template <typename V>
constexpr size_t agg_chunk_smem() { return (size_t)AGG_CH_SLOTS * (sizeof(V) + sizeof(int)) + (size_t)AGG_CH * sizeof(int); }

__global__ void k_agg_big_nchunks(int nbig, const int32_t* __restrict__ bigc, const long long* __restrict__ ent,
                                  long long* __restrict__ nch, int ch) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nbig; i += gridDim.x * blockDim.x)
        nch[i] = (ent[bigc[i]] + ch - 1) / ch;
}

template <bool UNIT, typename V>
__global__ void __launch_bounds__(256) k_agg_big_chunk(AggArgs a, const int32_t* __restrict__ bigc, int nbig,
                                                       const long long* __restrict__ choff,
                                                       const long long* __restrict__ goff, int* __restrict__ gkeys,
                                                       ull* __restrict__ gvals, int* __restrict__ glist,
                                                       int* __restrict__ gcnt, int ch) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    V* vals = reinterpret_cast<V*>(smem_raw);
    int* keys = reinterpret_cast<int*>(smem_raw + (size_t)AGG_CH_SLOTS * sizeof(V));
    int* list = keys + AGG_CH_SLOTS;
    __shared__ int s_cnt;
    __shared__ V s_scr[8][32];
    const int wib = threadIdx.x >> 5;
    for (int j = threadIdx.x; j < AGG_CH_SLOTS; j += 256) { keys[j] = -1; vals[j] = 0; }
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    const long long total = choff[nbig];
    for (long long t = blockIdx.x; t < total; t += gridDim.x) {
        const int bi = (int)seg_search(choff, 0, nbig - 1, t);
        const long long c = bigc[bi];
        const long long s1 = a.eoff[c + 1];
        const long long lo = a.eoff[c] + (t - choff[bi]) * ch;
        const long long hi = lo + ch < s1 ? lo + ch : s1;
        agg_segment<UNIT, V, V>(a, lo, hi, threadIdx.x, 256, keys, vals, AGG_CH_SLOTS - 1, list, &s_cnt, s_scr[wib]);
        __syncthreads();
        const int m = s_cnt;
        const long long off = goff[bi];
        const unsigned mask = (unsigned)(goff[bi + 1] - off) - 1u;
        for (int i0 = threadIdx.x & ~31; i0 < m; i0 += 256) {   // warp-uniform trips
            const int i = i0 + (threadIdx.x & 31);
            const bool on = i < m;
            int key = 0;
            V val = 0;
            if (on) {
                const int slot = list[i];
                key = keys[slot];
                val = vals[slot];
                keys[slot] = -1;
                vals[slot] = 0;
            }
            agg_insert_warp<ull>(on, key, (ull)val, gkeys + off, gvals + off, mask, glist + off / 2, &gcnt[bi]);
        }
        __syncthreads();
        if (threadIdx.x == 0) s_cnt = 0;
        __syncthreads();
    }
}

// Two-pass variant (option agg_bound, default): pass 1 combines every chunk in block smem and
// writes its distinct (key, sum) pairs back to the start of the chunk's own range of the
// segment (ndc[t] of them); the global table of a community is then sized from
// B = sum of its chunks' distinct counts (<= entries, usually far below), nextpow2(2 min(B, k))
// slots, and pass 2 inserts the chunk-distinct pairs.
template <bool UNIT, typename V>
__global__ void __launch_bounds__(256) k_agg_big_combine(AggArgs a, const int32_t* __restrict__ bigc, int nbig,
                                                         const long long* __restrict__ choff, int* __restrict__ ndc,
                                                         int ch) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    V* vals = reinterpret_cast<V*>(smem_raw);
    int* keys = reinterpret_cast<int*>(smem_raw + (size_t)AGG_CH_SLOTS * sizeof(V));
    int* list = keys + AGG_CH_SLOTS;
    __shared__ int s_cnt;
    __shared__ V s_scr[8][32];
    const int wib = threadIdx.x >> 5;
    for (int j = threadIdx.x; j < AGG_CH_SLOTS; j += 256) { keys[j] = -1; vals[j] = 0; }
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    const long long total = choff[nbig];
    for (long long t = blockIdx.x; t < total; t += gridDim.x) {
        const int bi = (int)seg_search(choff, 0, nbig - 1, t);
        const long long c = bigc[bi];
        const long long s1 = a.eoff[c + 1];
        const long long lo = a.eoff[c] + (t - choff[bi]) * ch;
        const long long hi = lo + ch < s1 ? lo + ch : s1;
        agg_segment<UNIT, V, V>(a, lo, hi, threadIdx.x, 256, keys, vals, AGG_CH_SLOTS - 1, list, &s_cnt, s_scr[wib]);
        __syncthreads();   // every entry of the chunk is read before its range is overwritten
        const int m = s_cnt;
        for (int i = threadIdx.x; i < m; i += 256) {
            const int slot = list[i];
            a.tkey[lo + i] = keys[slot];
            a.tval.set(lo + i, (int64_t)vals[slot]);
            keys[slot] = -1;
            vals[slot] = 0;
        }
        if (threadIdx.x == 0) ndc[t] = m;
        __syncthreads();
        if (threadIdx.x == 0) s_cnt = 0;
        __syncthreads();
    }
}

// table slots of big community i: nextpow2(2 min(B_i, k)), B_i = sum of its chunks' distinct counts
__global__ void k_agg_big_bound(int nbig, long long k, const long long* __restrict__ choff,
                                const int* __restrict__ ndc, long long* __restrict__ bigcap) {
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long i = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < nbig; i += nw) {
        long long b = 0;
        for (long long t = choff[i] + lane; t < choff[i + 1]; t += 32) b += ndc[t];
        b = warp_sum_ll(b);
        if (lane == 0) {
            const long long m = b < k ? b : k;
            bigcap[i] = m > 0 ? 1LL << (64 - __clzll(2 * m - 1)) : 1;
        }
    }
}

// GV: global table value type, 32-bit whenever W < 2^32 (halves the tables' value bytes)
template <typename GV>
__global__ void __launch_bounds__(256) k_agg_big_insert2(AggArgs a, const int32_t* __restrict__ bigc, int nbig,
                                                         const long long* __restrict__ choff,
                                                         const int* __restrict__ ndc, int ch,
                                                         const long long* __restrict__ goff, int* __restrict__ gkeys,
                                                         GV* __restrict__ gvals, int* __restrict__ glist,
                                                         int* __restrict__ gcnt) {
    const long long total = choff[nbig];
    for (long long t = blockIdx.x; t < total; t += gridDim.x) {
        const int bi = (int)seg_search(choff, 0, nbig - 1, t);
        const long long c = bigc[bi];
        const long long lo = a.eoff[c] + (t - choff[bi]) * ch;
        const int m = ndc[t];
        const long long off = goff[bi];
        const unsigned mask = (unsigned)(goff[bi + 1] - off) - 1u;
        for (int i0 = threadIdx.x & ~31; i0 < m; i0 += 256) {   // warp-uniform trips
            const int i = i0 + (threadIdx.x & 31);
            const bool on = i < m;
            agg_insert_warp<GV>(on, on ? a.tkey[lo + i] : 0, on ? (GV)a.tval.get(lo + i) : (GV)0, gkeys + off, gvals + off, mask,
                            glist + off / 2, &gcnt[bi]);
        }
    }
}

// distinct entries of the big communities to the start of their segments; list
// index range of chunk t = [j*AGG_CH, (j+1)*AGG_CH) of its community (m <= entries)
template <typename GV>
__global__ void __launch_bounds__(256) k_agg_big_emit2(AggArgs a, const int32_t* __restrict__ bigc, int nbig,
                                                       const long long* __restrict__ choff,
                                                       const long long* __restrict__ goff,
                                                       const int* __restrict__ gkeys, const GV* __restrict__ gvals,
                                                       const int* __restrict__ glist, const int* __restrict__ gcnt,
                                                       int ch) {
    const long long total = choff[nbig];
    for (long long t = blockIdx.x; t < total; t += gridDim.x) {
        const int bi = (int)seg_search(choff, 0, nbig - 1, t);
        const long long c = bigc[bi];
        const long long off = goff[bi];
        const int m = gcnt[bi];
        const long long j = t - choff[bi];
        const int lo = (int)(j * ch);
        const int hi = lo + ch < m ? lo + ch : m;
        const long long o = a.eoff[c];
        const int* list = glist + off / 2;
        for (int i = lo + threadIdx.x; i < hi; i += 256) {
            const int slot = list[i];
            const int key = gkeys[off + slot];
            const int64_t val = (int64_t)gvals[off + slot];
            a.tkey[o + i] = key;
            a.tval.set(o + i, val);
            if (key == (int)c) a.snew[c] = val;
        }
        if (j == 0 && threadIdx.x == 0) a.dn[c] = m;
    }
}

// thread per coarse entry t: row c = segment of t in rp_new (bounded search per
// 256-entry block), copy from the aggregated segment at eoff[c]
// tile map for k_compact: tmap[t] = the community whose coarse row holds entry 256*t
__global__ void k_tile_map(long long k, const long long* __restrict__ rp_new, long long nnz_new,
                           int32_t* __restrict__ tmap) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < k; c += (long long)gridDim.x * blockDim.x) {
        const long long a = rp_new[c], b = rp_new[c + 1];
        for (long long t = (a + 255) & ~255LL; t < b; t += 256) tmap[t >> 8] = (int32_t)c;
    }
}

// thread per coarse entry t: row c = segment of t in rp_new, searched between the
// communities of this tile's start and the next tile's start (tile map), copy
// from the aggregated segment at eoff[c]
__global__ void __launch_bounds__(256) k_compact(long long k, long long nnz_new, const long long* __restrict__ eoff,
                                                 const long long* __restrict__ rp_new, const int32_t* __restrict__ tmap,
                                                 const int* __restrict__ tkey, TVal tval,
                                                 int32_t* __restrict__ col_new, int64_t* __restrict__ w_new,
                                                 int32_t* __restrict__ row_new) {
    const long long ntiles = (nnz_new + 255) >> 8;
    for (long long tb = blockIdx.x; tb < ntiles; tb += gridDim.x) {
        const long long lo = tmap[tb];
        const long long hi = tb + 1 < ntiles ? tmap[tb + 1] : k - 1;
        const long long t = (tb << 8) + threadIdx.x;
        if (t < nnz_new) {
            const long long c = seg_search(rp_new, lo, hi, t);
            const long long src = eoff[c] + (t - rp_new[c]);
            col_new[t] = tkey[src];
            w_new[t] = tval.get(src);
            row_new[t] = (int32_t)c;
        }
    }
}

// coarse d(c') = Sigma_tot of the community (maintained exactly by phase 1)
__global__ void k_coarsen_deg(int n, const int32_t* __restrict__ C, const int32_t* __restrict__ minmem,
                              const int32_t* __restrict__ newid, const int64_t* __restrict__ Sig,
                              int64_t* __restrict__ d_new) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
        if (minmem[C[v]] == v) d_new[newid[v]] = Sig[C[v]];
}

// input validation on the device: flags |= 1 row_ptr decreasing, 2 column out of
// range, 4 weight <= 0, 8 some weight != 1
__global__ void k_validate(int n, long long nnz, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                           const int64_t* __restrict__ w, unsigned* __restrict__ flags) {
    unsigned f = 0;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
        if (rp[v + 1] < rp[v]) f |= 1u;
    for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += stride) {
        int c = col[e];
        if (c < 0 || c >= n) f |= 2u;
        if (w) {
            long long x = w[e];
            if (x <= 0) f |= 4u;
            if (x != 1) f |= 8u;
        }
    }
    f = __reduce_or_sync(FULLMASK, f);
    if (lane_id() == 0 && f) atomicOr(flags, f);
}

// sum of a non-negative int64 array as int128 (per-block partials + last block)
__global__ void __launch_bounds__(256) k_sum_i128(long long n, const int64_t* __restrict__ x, i128* __restrict__ part,
                                                  ull* __restrict__ ticket, i128* __restrict__ out) {
    __shared__ i128 sh[8];
    __shared__ bool amLast;
    i128 s = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        s += (i128)x[i];
    for (int o = 16; o > 0; o >>= 1) s += shfl_xor_st(s, o);
    if (lane_id() == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < (int)(blockDim.x >> 5); ++i) s += sh[i];
        part[blockIdx.x] = s;
        __threadfence();
        amLast = atomicAdd(ticket, 1ull) == gridDim.x - 1;
    }
    __syncthreads();
    if (amLast && threadIdx.x == 0) {
        __threadfence();
        i128 t = 0;
        for (int b = 0; b < (int)gridDim.x; ++b) t += part[b];
        *out = t;
        *ticket = 0;
    }
}

// *bad != 0 iff some row is not strictly increasing (so may hold duplicate columns)
// entries that do not strictly increase within their row (duplicates / unsorted rows), edge-parallel
// over the row-id array (a thread per row walked the longest rows -- 33k entries -- serially)
__global__ void k_rows_not_increasing(long long nnz, const int32_t* __restrict__ row, const int32_t* __restrict__ col,
                                      ull* __restrict__ bad) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    unsigned f = 0;
    for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x + 1; e < nnz; e += stride)
        if (row[e] == row[e - 1] && col[e] <= col[e - 1]) f = 1;
    f = __reduce_or_sync(FULLMASK, f);
    if (lane_id() == 0 && f) atomicAdd(bad, 1ull);
}

// max of a non-negative int64 array
__global__ void k_max_i64(long long n, const int64_t* __restrict__ x, ull* __restrict__ out) {
    ull m = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        m = (ull)x[i] > m ? (ull)x[i] : m;
    for (int o = 16; o > 0; o >>= 1) {
        ull y = __shfl_xor_sync(FULLMASK, m, o);
        m = y > m ? y : m;
    }
    if (lane_id() == 0 && m) atomicMax(out, m);
}

// max row length of the coarse graph
__global__ void k_rowmax(long long k, const long long* __restrict__ rp, ull* __restrict__ out) {
    ull m = 0;
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < k; c += (long long)gridDim.x * blockDim.x) {
        ull x = (ull)(rp[c + 1] - rp[c]);
        m = x > m ? x : m;
    }
    for (int o = 16; o > 0; o >>= 1) {
        ull y = __shfl_xor_sync(FULLMASK, m, o);
        m = y > m ? y : m;
    }
    if (lane_id() == 0 && m) atomicMax(out, m);
}

// ---------------------------------------------------------------------------
// final modularity numerator on the level-0 graph from the composed labels
// (Eq. 1): DC = sum of entries with both ends in one community; DV[c] += d(v)
// ---------------------------------------------------------------------------
template <bool UNIT>
__global__ void __launch_bounds__(256) k_mod_dc(int n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                const int64_t* __restrict__ w, const int32_t* __restrict__ lab,
                                                const int64_t* __restrict__ d, long long* __restrict__ DV,
                                                ull* __restrict__ DC) {
    const int lane = lane_id();
    long long wid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    long long acc = 0;
    for (long long v = wid; v < n; v += nw) {
        int lv = lab[v];
        for (int64_t j = rp[v] + lane; j < rp[v + 1]; j += 32)
            if (lab[col[j]] == lv) acc += UNIT ? 1 : w[j];
        if (lane == 0 && d[v]) atomicAdd(reinterpret_cast<ull*>(&DV[lv]), (ull)d[v]);
    }
    acc = warp_sum_ll(acc);
    if (lane == 0 && acc) atomicAdd(DC, (ull)acc);
}

// sum of DV[c]^2 (int128) via per-block partials + last block
__global__ void __launch_bounds__(256) k_sumsq(long long n, const long long* __restrict__ x, i128* __restrict__ part,
                                               ull* __restrict__ ticket, i128* __restrict__ out) {
    __shared__ i128 sh[8];
    __shared__ bool amLast;
    i128 s = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        s += (i128)x[i] * x[i];
    for (int o = 16; o > 0; o >>= 1) s += shfl_xor_st(s, o);
    if (lane_id() == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < (int)(blockDim.x >> 5); ++i) s += sh[i];
        part[blockIdx.x] = s;
        __threadfence();
        amLast = atomicAdd(ticket, 1ull) == gridDim.x - 1;
    }
    __syncthreads();
    if (amLast && threadIdx.x == 0) {
        __threadfence();
        i128 t = 0;
        for (int b = 0; b < (int)gridDim.x; ++b) t += part[b];
        *out = t;
        *ticket = 0;
    }
}
