// k_phase1.cuh — phase-1 kernels (Alg. 1): level init, MG pruning
// frontier + degree binning, DecideAndMove (sub-warp shuffle, warp hash,
// block hierarchical hash), apply moves, d' update, Q/convergence reduction.
// SURVEY.md §8(a) rows a1-a7; DESIGN.md "Kernels".
#pragma once
#include "common.cuh"

// ---------------------------------------------------------------------------
// a1: weighted degree d(v) and self-loop weight s(v) of every vertex (warp per row)
// ---------------------------------------------------------------------------
template <bool UNIT>
__global__ void k_degrees(int n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                          const int64_t* __restrict__ w, int64_t* __restrict__ d, int64_t* __restrict__ s,
                          ull* __restrict__ maxdeg) {
    const int lane = lane_id();
    long long wid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    ull mymax = 0;
    for (long long v = wid; v < n; v += nw) {
        int64_t b = rp[v], e = rp[v + 1];
        long long dv = 0, sv = 0;
        for (int64_t j = b + lane; j < e; j += 32) {
            long long x = UNIT ? 1 : w[j];
            dv += x;
            if (col[j] == v) sv += x;
        }
        dv = warp_sum_ll(dv);
        sv = warp_sum_ll(sv);
        if (lane == 0) {
            d[v] = dv;
            s[v] = sv;
            if ((ull)(e - b) > mymax) mymax = (ull)(e - b);
        }
    }
    if (lane == 0 && mymax) atomicMax(maxdeg, mymax);
}

// a1: every vertex its own community
__global__ void k_level_init(int n, const int64_t* __restrict__ d, int32_t* __restrict__ C,
                             int64_t* __restrict__ Sig, int32_t* __restrict__ size, int64_t* __restrict__ dp,
                             int32_t* __restrict__ stamp) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n;
         v += (long long)gridDim.x * blockDim.x) {
        C[v] = (int32_t)v;
        Sig[v] = d[v];
        size[v] = 1;
        dp[v] = 0;
        stamp[v] = -1;
    }
}

__global__ void k_iter_begin(IterCounters* ctr) {
    ull* p = reinterpret_cast<ull*>(ctr);
    for (int i = threadIdx.x; i < (int)(sizeof(IterCounters) / sizeof(ull)); i += blockDim.x) p[i] = 0;
}

// ---------------------------------------------------------------------------
// a2: MG pruning frontier (Eq. 6/7) fused with degree binning.
//   inactive iff  qW (2 d'(v) - d(v)) + p (minSig - Sig[C[v]]) d(v) >= 0
// Active vertices are appended to the queue of their degree bin with
// warp-aggregated atomics.  Bin choice never changes results (P7).
// ---------------------------------------------------------------------------
struct BinThresholds {
    int t[NBINS - 1];   // upper row-length bound of bins 0..4; bin 5 = rest
};

template <typename ST>
__global__ void __launch_bounds__(256) k_prune_bin(int n, const int64_t* __restrict__ rp,
                                                   const int64_t* __restrict__ d, const int64_t* __restrict__ dp,
                                                   const int32_t* __restrict__ C, const int64_t* __restrict__ Sig,
                                                   int prune, ST qW, ST p, const Carry* __restrict__ carry,
                                                   IterCounters* __restrict__ ctr, int32_t* __restrict__ queues,
                                                   long long qstride, BinThresholds th) {
    const long long minSig = carry->minSig;
    ull my_active = 0, my_pruned = 0;
    ull my_deg[NBINS] = {0, 0, 0, 0, 0, 0};
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long base = (long long)blockIdx.x * blockDim.x; base < n; base += stride) {
        long long v = base + threadIdx.x;
        int bin = -1;
        int deg = 0;
        if (v < n) {
            long long dv = d[v];
            if (dv > 0) {
                bool active = true;
                if (prune) {
                    long long dpv = dp[v];
                    long long sg = Sig[C[v]];
                    ST lhs = qW * (ST)(2 * dpv - dv) + p * (ST)(minSig - sg) * (ST)dv;
                    active = lhs < (ST)0;
                }
                if (active) {
                    long long dg = rp[v + 1] - rp[v];
                    deg = (int)(dg > INT_MAX ? INT_MAX : dg);
                    bin = NBINS - 1;
#pragma unroll
                    for (int b = NBINS - 2; b >= 0; --b)
                        if (deg <= th.t[b]) bin = b;
                    my_active++;
                } else {
                    my_pruned++;
                }
            }
        }
        // warp-aggregated append per bin
        unsigned peers = __match_any_sync(FULLMASK, bin);
        int leader = __ffs(peers) - 1;
        ull basepos = 0;
        if (bin >= 0 && lane_id() == leader) basepos = atomicAdd(&ctr->bin_count[bin], (ull)__popc(peers));
        basepos = __shfl_sync(FULLMASK, basepos, leader);
        if (bin >= 0) {
            long long pos = (long long)basepos + __popc(peers & lanemask_lt());
            queues[(long long)bin * qstride + pos] = (int32_t)v;
#pragma unroll
            for (int b = 0; b < NBINS; ++b)
                if (b == bin) my_deg[b] += (ull)deg;
        }
    }
    // counters (one atomic per warp)
    ull a = __reduce_add_sync(FULLMASK, (unsigned)my_active);
    ull pr = __reduce_add_sync(FULLMASK, (unsigned)my_pruned);
    if (lane_id() == 0) {
        if (a) atomicAdd(&ctr->n_active, a);
        if (pr) atomicAdd(&ctr->n_pruned, pr);
    }
#pragma unroll
    for (int b = 0; b < NBINS; ++b) {
        ull x = my_deg[b];
        for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(FULLMASK, x, o);
        if (lane_id() == 0 && x) atomicAdd(&ctr->bin_deg[b], x);
    }
}

// ---------------------------------------------------------------------------
// decision shared by all DecideAndMove kernels
// ---------------------------------------------------------------------------
template <typename ST>
__device__ __forceinline__ int decide_final(int cv, long long dv, long long own, ST best_s, int best_c,
                                            const int64_t* __restrict__ Sig, const int32_t* __restrict__ size,
                                            ST qW, ST p) {
    ST stay = qW * (ST)own - p * (ST)(Sig[cv] - dv) * (ST)dv;
    int tgt = cv;
    if (best_c != INT_MAX && best_s > stay) {          // strictly better than staying (c4)
        tgt = best_c;
        if (size[tgt] == 1 && size[cv] == 1 && tgt > cv) tgt = cv;   // swap suppression (c5)
    }
    return tgt;
}

struct DecideArgs {
    const int64_t* rp;
    const int32_t* col;
    const int64_t* w;
    const int32_t* C;
    const int64_t* Sig;
    const int32_t* size;
    const int64_t* d;
    const int64_t* dp;
    int32_t* mv_v;      // moved list: vertex
    int32_t* mv_c;      // moved list: target community
    IterCounters* ctr;
    int check;
};

// ---------------------------------------------------------------------------
// a3: low-degree DecideAndMove — sub-warp groups of G lanes, one neighbour per
// lane, community aggregation with __match_any_sync (Alg. 2).
// Weighted levels sum the peers' weights with shared-memory atomics onto the
// group leader; unit-weight levels use popc(peers).  Argmax over the group
// with an xor-shuffle butterfly on (score, -community).
// ---------------------------------------------------------------------------
template <int G, typename ST, bool UNIT>
__global__ void __launch_bounds__(256) k_decide_sub(const int32_t* __restrict__ queue, int bin, DecideArgs a,
                                                    ST qW, ST p) {
    __shared__ ull s_acc[8][32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const int gid = lane / G, gl = lane % G;
    const unsigned gmask = (G == 32) ? FULLMASK : (((1u << G) - 1u) << (gid * G));
    const long long count = (long long)a.ctr->bin_count[bin];
    const long long nwarps = (long long)gridDim.x * (blockDim.x >> 5);
    const long long per = 32 / G;
    ull my_k = 0, my_moved_deg = 0;
    for (long long base = ((long long)blockIdx.x * (blockDim.x >> 5) + wib) * per; base < count;
         base += nwarps * per) {
        long long i = base + gid;
        bool valid = i < count;
        int v = valid ? queue[i] : 0;
        int64_t beg = valid ? a.rp[v] : 0;
        int deg = valid ? (int)(a.rp[v + 1] - beg) : 0;
        bool has = valid && gl < deg;
        int u = has ? a.col[beg + gl] : -1;
        if (u == v) has = false;                          // self loop is not a neighbour
        long long wt = has ? (UNIT ? 1 : a.w[beg + gl]) : 0;
        int cu = has ? a.C[u] : (-1 - lane);              // unique sentinel per empty lane
        unsigned peers = __match_any_sync(FULLMASK, cu) & gmask;
        int leader = __ffs(peers) - 1;
        bool isL = has && lane == leader;
        long long wc;
        if (UNIT) {
            wc = __popc(peers);
        } else {
            s_acc[wib][lane] = 0;
            __syncwarp();
            if (has) atomicAdd(&s_acc[wib][leader], (ull)wt);
            __syncwarp();
            wc = (long long)s_acc[wib][lane];
            __syncwarp();
        }
        int cv = valid ? a.C[v] : -2;
        long long dv = valid ? a.d[v] : 0;
        ST bs = st_min<ST>();
        int bc = INT_MAX;
        long long own = 0;
        if (isL) {
            my_k++;
            if (cu == cv) own = wc;
            else { bs = qW * (ST)wc - p * (ST)a.Sig[cu] * (ST)dv; bc = cu; }
        }
#pragma unroll
        for (int off = G / 2; off > 0; off >>= 1) {
            ST os = shfl_xor_st(bs, off);
            int oc = __shfl_xor_sync(FULLMASK, bc, off);
            own += __shfl_xor_sync(FULLMASK, own, off);
            if (better(os, oc, bs, bc)) { bs = os; bc = oc; }
        }
        int tgt = cv;
        if (valid && gl == 0) {
            if (a.check && own != a.dp[v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            if (dv > 0) tgt = decide_final<ST>(cv, dv, own, bs, bc, a.Sig, a.size, qW, p);
        }
        bool mover = valid && gl == 0 && tgt != cv;
        long long pos = warp_append(mover, &a.ctr->n_moved);
        if (mover) {
            a.mv_v[pos] = v;
            a.mv_c[pos] = tgt;
            my_moved_deg += (ull)deg;
        }
    }
    ull k = __reduce_add_sync(FULLMASK, (unsigned)my_k);
    ull md = __reduce_add_sync(FULLMASK, (unsigned)my_moved_deg);
    if (lane == 0) {
        if (k) atomicAdd(&a.ctr->bin_k[bin], k);
        if (md) atomicAdd(&a.ctr->moved_deg, md);
    }
}

// ---------------------------------------------------------------------------
// open-addressing insert: (key, +w) with CAS on the key, atomicAdd on the value
// (Alg. 3 lines 6-10).  Linear probing up to `win` slots; returns false
// if the window is full of other keys.
// ---------------------------------------------------------------------------
__device__ __forceinline__ bool ht_insert(int c, ull wt, int* keys, ull* vals, unsigned mask, unsigned h,
                                          int win) {
    for (int t = 0; t < win; ++t) {
        int k = *(volatile int*)&keys[h];
        if (k == -1) {
            int old = atomicCAS(&keys[h], -1, c);
            if (old == -1 || old == c) { atomicAdd(&vals[h], wt); return true; }
        } else if (k == c) {
            atomicAdd(&vals[h], wt);
            return true;
        }
        h = (h + 1) & mask;
    }
    return false;
}

// ---------------------------------------------------------------------------
// a4 (mid degree): one warp per vertex, per-warp shared-memory hash table with
// capacity nextpow2(2 deg) <= WCAP (load factor <= 1/2, never spills).
// ---------------------------------------------------------------------------
template <int WCAP, typename ST, bool UNIT>
__global__ void __launch_bounds__(256) k_decide_warp(const int32_t* __restrict__ queue, int bin, DecideArgs a,
                                                     ST qW, ST p) {
    __shared__ int s_key[8][WCAP];
    __shared__ ull s_val[8][WCAP];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    int* keys = s_key[wib];
    ull* vals = s_val[wib];
    const long long count = (long long)a.ctr->bin_count[bin];
    const long long nwarps = (long long)gridDim.x * (blockDim.x >> 5);
    ull my_k = 0;
    for (long long i = (long long)blockIdx.x * (blockDim.x >> 5) + wib; i < count; i += nwarps) {
        int v = queue[i];
        int64_t beg = a.rp[v];
        int deg = (int)(a.rp[v + 1] - beg);
        int cap = 64;
        while (cap < 2 * deg && cap < WCAP) cap <<= 1;
        unsigned mask = (unsigned)cap - 1;
        for (int j = lane; j < cap; j += 32) { keys[j] = -1; vals[j] = 0; }
        __syncwarp();
        for (int j = lane; j < deg; j += 32) {
            int u = a.col[beg + j];
            if (u == v) continue;
            ull wt = UNIT ? 1ull : (ull)a.w[beg + j];
            int c = a.C[u];
            ht_insert(c, wt, keys, vals, mask, hash_slot(c, mask), cap);
        }
        __syncwarp();
        int cv = a.C[v];
        long long dv = a.d[v];
        ST bs = st_min<ST>();
        int bc = INT_MAX;
        long long own = 0;
        for (int j = lane; j < cap; j += 32) {
            int c = keys[j];
            if (c < 0) continue;
            my_k++;
            long long wc = (long long)vals[j];
            if (c == cv) { own = wc; continue; }
            ST sc = qW * (ST)wc - p * (ST)a.Sig[c] * (ST)dv;
            if (better(sc, c, bs, bc)) { bs = sc; bc = c; }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
            ST os = shfl_xor_st(bs, off);
            int oc = __shfl_xor_sync(FULLMASK, bc, off);
            own += __shfl_xor_sync(FULLMASK, own, off);
            if (better(os, oc, bs, bc)) { bs = os; bc = oc; }
        }
        if (lane == 0) {
            if (a.check && own != a.dp[v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            int tgt = decide_final<ST>(cv, dv, own, bs, bc, a.Sig, a.size, qW, p);
            if (tgt != cv) {
                ull pos = atomicAdd(&a.ctr->n_moved, 1ull);
                a.mv_v[pos] = v;
                a.mv_c[pos] = tgt;
                atomicAdd(&a.ctr->moved_deg, (ull)deg);
            }
        }
        __syncwarp();
    }
    ull k = __reduce_add_sync(FULLMASK, (unsigned)my_k);
    if (lane == 0 && k) atomicAdd(&a.ctr->bin_k[bin], k);
}

// ---------------------------------------------------------------------------
// a4 (high degree / hubs): one block per vertex, hierarchical hash table
// (§4.2 "Hierarchical"): shared-memory table H0 probed first
// (window of HWIN slots), overflow to a per-block global table H1 with linear
// probing.  H1 is left clean (all empty) after every vertex: the scan phase
// resets the slots it reads.  Vertices are fetched dynamically.
// ---------------------------------------------------------------------------
#define HWIN 16
template <int BT, typename ST, bool UNIT>
__global__ void __launch_bounds__(BT) k_decide_block(const int32_t* __restrict__ queue, int bin, DecideArgs a,
                                                     ST qW, ST p, int smem_cap, int* __restrict__ gkeys_all,
                                                     ull* __restrict__ gvals_all, long long gcap) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    ull* vals = reinterpret_cast<ull*>(smem_raw);
    int* keys = reinterpret_cast<int*>(smem_raw + (size_t)smem_cap * sizeof(ull));
    __shared__ long long s_item;
    __shared__ int s_spill;
    __shared__ ST r_s[BT / 32];
    __shared__ int r_c[BT / 32];
    __shared__ long long r_own[BT / 32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    int* gkeys = gkeys_all + (long long)blockIdx.x * gcap;
    ull* gvals = gvals_all + (long long)blockIdx.x * gcap;
    const long long count = (long long)a.ctr->bin_count[bin];
    ull my_k = 0;
    for (;;) {
        if (threadIdx.x == 0) {
            s_item = (long long)atomicAdd(&a.ctr->cursor[bin], 1ull);
            s_spill = 0;
        }
        __syncthreads();
        long long i = s_item;
        if (i >= count) break;
        int v = queue[i];
        int64_t beg = a.rp[v];
        int deg = (int)(a.rp[v + 1] - beg);
        int cap = 64;
        while (cap < 2 * deg && cap < smem_cap) cap <<= 1;
        unsigned mask = (unsigned)cap - 1;
        int win = (cap >= 2 * deg) ? cap : HWIN;      // fits: plain linear probing, never spills
        long long gc = 64;
        while (gc < 2LL * deg && gc < gcap) gc <<= 1;
        unsigned gmask = (unsigned)gc - 1;
        for (int j = threadIdx.x; j < cap; j += BT) { keys[j] = -1; vals[j] = 0; }
        __syncthreads();
        for (int j = threadIdx.x; j < deg; j += BT) {
            int u = a.col[beg + j];
            if (u == v) continue;
            ull wt = UNIT ? 1ull : (ull)a.w[beg + j];
            int c = a.C[u];
            if (!ht_insert(c, wt, keys, vals, mask, hash_slot(c, mask), win)) {
                if (!s_spill) s_spill = 1;
                ht_insert(c, wt, gkeys, gvals, gmask, hash_slot2(c, gmask), (int)gc);
            }
        }
        __syncthreads();
        int cv = a.C[v];
        long long dv = a.d[v];
        ST bs = st_min<ST>();
        int bc = INT_MAX;
        long long own = 0;
        for (int j = threadIdx.x; j < cap; j += BT) {
            int c = keys[j];
            if (c < 0) continue;
            my_k++;
            long long wc = (long long)vals[j];
            if (c == cv) { own = wc; continue; }
            ST sc = qW * (ST)wc - p * (ST)a.Sig[c] * (ST)dv;
            if (better(sc, c, bs, bc)) { bs = sc; bc = c; }
        }
        if (s_spill) {
            for (long long j = threadIdx.x; j < gc; j += BT) {
                int c = gkeys[j];
                if (c < 0) continue;
                my_k++;
                long long wc = (long long)gvals[j];
                gkeys[j] = -1;
                gvals[j] = 0;
                if (c == cv) { own = wc; continue; }
                ST sc = qW * (ST)wc - p * (ST)a.Sig[c] * (ST)dv;
                if (better(sc, c, bs, bc)) { bs = sc; bc = c; }
            }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
            ST os = shfl_xor_st(bs, off);
            int oc = __shfl_xor_sync(FULLMASK, bc, off);
            own += __shfl_xor_sync(FULLMASK, own, off);
            if (better(os, oc, bs, bc)) { bs = os; bc = oc; }
        }
        if (lane == 0) { r_s[wib] = bs; r_c[wib] = bc; r_own[wib] = own; }
        __syncthreads();
        if (wib == 0) {
            bs = lane < BT / 32 ? r_s[lane] : st_min<ST>();
            bc = lane < BT / 32 ? r_c[lane] : INT_MAX;
            own = lane < BT / 32 ? r_own[lane] : 0;
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) {
                ST os = shfl_xor_st(bs, off);
                int oc = __shfl_xor_sync(FULLMASK, bc, off);
                own += __shfl_xor_sync(FULLMASK, own, off);
                if (better(os, oc, bs, bc)) { bs = os; bc = oc; }
            }
            if (lane == 0) {
                if (a.check && own != a.dp[v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
                int tgt = decide_final<ST>(cv, dv, own, bs, bc, a.Sig, a.size, qW, p);
                if (tgt != cv) {
                    ull pos = atomicAdd(&a.ctr->n_moved, 1ull);
                    a.mv_v[pos] = v;
                    a.mv_c[pos] = tgt;
                    atomicAdd(&a.ctr->moved_deg, (ull)deg);
                }
            }
        }
        __syncthreads();   // table reuse / s_item
    }
    ull k = __reduce_add_sync(FULLMASK, (unsigned)my_k);
    if (lane == 0 && k) atomicAdd(&a.ctr->bin_k[bin], k);
}

// ---------------------------------------------------------------------------
// a5: apply moves (Alg. 1 line 5): Sigma_tot and sizes by int atomics
// (order-independent), C[v] <- new, remember the old community for a6.
// ---------------------------------------------------------------------------
__global__ void k_apply(IterCounters* __restrict__ ctr, const int32_t* __restrict__ mv_v,
                        const int32_t* __restrict__ mv_c, int32_t* __restrict__ mv_old, int32_t* __restrict__ C,
                        int64_t* __restrict__ Sig, int32_t* __restrict__ size, const int64_t* __restrict__ d,
                        int32_t* __restrict__ stamp, int iter_id) {
    const long long m = (long long)ctr->n_moved;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (long long)gridDim.x * blockDim.x) {
        int v = mv_v[i], nc = mv_c[i];
        int oc = C[v];
        long long dv = d[v];
        mv_old[i] = oc;
        C[v] = nc;
        stamp[v] = iter_id;
        atomicAdd(reinterpret_cast<ull*>(&Sig[oc]), (ull)(-dv));
        atomicAdd(reinterpret_cast<ull*>(&Sig[nc]), (ull)dv);
        atomicSub(&size[oc], 1);
        atomicAdd(&size[nc], 1);
    }
}

// ---------------------------------------------------------------------------
// a6: community-weight update (§3.5).
// Delta form, warp per moved vertex u: recompute d'(u) from its row (C is
// already updated) and push -w / +w to every UNMOVED neighbour x whose
// community is u's old / new one.  Selected on the device when the moved
// volume is small; otherwise k_dp_full recomputes d' for every vertex.
// ---------------------------------------------------------------------------
__device__ __forceinline__ bool use_delta(const IterCounters* ctr, long long nnz, int mode, long long frac_num,
                                          long long frac_den) {
    if (mode == 0) return false;
    if (mode == 1) return true;
    return (long long)ctr->moved_deg * frac_den <= nnz * frac_num;
}

template <bool UNIT>
__global__ void __launch_bounds__(256) k_dp_delta(IterCounters* __restrict__ ctr, const int64_t* __restrict__ rp,
                                                  const int32_t* __restrict__ col, const int64_t* __restrict__ w,
                                                  const int32_t* __restrict__ C, const int32_t* __restrict__ mv_v,
                                                  const int32_t* __restrict__ mv_old,
                                                  const int32_t* __restrict__ stamp, int64_t* __restrict__ dp,
                                                  int iter_id, long long nnz, int mode, long long fnum,
                                                  long long fden) {
    if (!use_delta(ctr, nnz, mode, fnum, fden)) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) ctr->delta_used = 1;
    const int lane = lane_id();
    const long long m = (long long)ctr->n_moved;
    long long wid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long i = wid; i < m; i += nw) {
        int u = mv_v[i], oc = mv_old[i];
        int nc = C[u];
        int64_t b = rp[u], e = rp[u + 1];
        long long acc = 0;
        for (int64_t j = b + lane; j < e; j += 32) {
            int x = col[j];
            if (x == u) continue;
            long long wt = UNIT ? 1 : w[j];
            int cx = C[x];
            if (cx == nc) acc += wt;
            if (stamp[x] != iter_id) {
                if (cx == oc) atomicAdd(reinterpret_cast<ull*>(&dp[x]), (ull)(-wt));
                else if (cx == nc) atomicAdd(reinterpret_cast<ull*>(&dp[x]), (ull)wt);
            }
        }
        acc = warp_sum_ll(acc);
        if (lane == 0) dp[u] = acc;
    }
}

// d'(v) = sum of w(v,u), u != v, C[u] == C[v]   (definition; 8 lanes per vertex)
template <bool UNIT>
__global__ void __launch_bounds__(256) k_dp_full(IterCounters* __restrict__ ctr, int n,
                                                 const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                 const int64_t* __restrict__ w, const int32_t* __restrict__ C,
                                                 int64_t* __restrict__ dp, long long nnz, int mode, long long fnum,
                                                 long long fden, int force) {
    if (!force && use_delta(ctr, nnz, mode, fnum, fden)) return;
    const int lane = lane_id(), gl = lane & 7;
    const long long ngroups = ((long long)gridDim.x * blockDim.x) >> 3;
    for (long long base = ((long long)blockIdx.x * blockDim.x + (threadIdx.x & ~31)) >> 3; base < n;
         base += ngroups) {
        long long v = base + (lane >> 3);
        long long acc = 0;
        if (v < n) {
            int cv = C[v];
            int64_t b = rp[v], e = rp[v + 1];
            for (int64_t j = b + gl; j < e; j += 8) {
                int x = col[j];
                if (x != v && C[x] == cv) acc += UNIT ? 1 : w[j];
            }
        }
        acc += __shfl_xor_sync(FULLMASK, acc, 4);
        acc += __shfl_xor_sync(FULLMASK, acc, 2);
        acc += __shfl_xor_sync(FULLMASK, acc, 1);
        if (v < n && gl == 0) dp[v] = acc;
    }
}

// ---------------------------------------------------------------------------
// a7: sumDC = sum_v (d'(v) + s(v)), S2 = sum_c Sig[c]^2 (int128), minSig =
// min{Sig > 0} (Alg. 1 lines 8-11).  N' = qW sumDC - p S2.  The last block
// to finish combines the per-block partials and takes the convergence
// decision dN < T (Alg. 1 lines 12-13) on the device.
// mode 0: level start (N := N'), mode 1: iteration end.
// ---------------------------------------------------------------------------
template <int BT>
__global__ void __launch_bounds__(BT) k_reduce(int n, const int64_t* __restrict__ dp, const int64_t* __restrict__ s,
                                               const int64_t* __restrict__ Sig, long long* __restrict__ part_dc,
                                               i128* __restrict__ part_s2, long long* __restrict__ part_min,
                                               IterCounters* __restrict__ ctr, Carry* __restrict__ carry,
                                               long long qW_hi, ull qW_lo, long long p, long long T_hi, ull T_lo,
                                               int mode) {
    __shared__ long long sh_dc[BT / 32];
    __shared__ i128 sh_s2[BT / 32];
    __shared__ long long sh_min[BT / 32];
    __shared__ bool amLast;
    long long dc = 0, mn = LLONG_MAX;
    i128 s2 = 0;
    for (long long v = (long long)blockIdx.x * BT + threadIdx.x; v < n; v += (long long)gridDim.x * BT) {
        dc += dp[v] + s[v];
        long long sg = Sig[v];
        s2 += (i128)sg * sg;
        if (sg > 0 && sg < mn) mn = sg;
    }
    const int lane = lane_id(), wib = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        dc += __shfl_xor_sync(FULLMASK, dc, o);
        s2 += shfl_xor_st(s2, o);
        long long om = __shfl_xor_sync(FULLMASK, mn, o);
        mn = om < mn ? om : mn;
    }
    if (lane == 0) { sh_dc[wib] = dc; sh_s2[wib] = s2; sh_min[wib] = mn; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < BT / 32; ++i) {
            dc += sh_dc[i];
            s2 += sh_s2[i];
            mn = sh_min[i] < mn ? sh_min[i] : mn;
        }
        part_dc[blockIdx.x] = dc;
        part_s2[blockIdx.x] = s2;
        part_min[blockIdx.x] = mn;
        __threadfence();
        ull t = atomicAdd(&ctr->ticket, 1ull);
        amLast = (t == gridDim.x - 1);
    }
    __syncthreads();
    if (amLast && threadIdx.x == 0) {
        __threadfence();
        long long tdc = 0, tmn = LLONG_MAX;
        i128 ts2 = 0;
        for (int b = 0; b < (int)gridDim.x; ++b) {
            tdc += *(volatile long long*)&part_dc[b];
            ts2 += part_s2[b];
            long long m2 = *(volatile long long*)&part_min[b];
            tmn = m2 < tmn ? m2 : tmn;
        }
        i128 qW = mk128(qW_hi, qW_lo);
        i128 Nn = qW * (i128)tdc - (i128)p * ts2;
        i128 N = mk128(carry->N_hi, carry->N_lo);
        int conv = 0;
        if (mode == 1) {
            i128 T = mk128(T_hi, T_lo);
            conv = (ctr->n_moved == 0) || (Nn - N < T);
        }
        carry->N_prev_hi = hi128(N);
        carry->N_prev_lo = lo128(N);
        carry->N_hi = hi128(Nn);
        carry->N_lo = lo128(Nn);
        carry->minSig = tmn;
        carry->sumDC = tdc;
        carry->converged = conv;
        ctr->ticket = 0;
    }
}
