// k_phase1.cuh — phase-1 kernels (Alg. 1): level init, MG pruning
// frontier + degree binning, DecideAndMove (sub-warp shuffle, warp hash,
// block hierarchical hash), apply moves, d' update, Q/convergence reduction,
// per-iteration device log.  SURVEY.md §8(a) rows a1-a7; DESIGN.md "Kernels".
//
// Throughput notes: the decide kernels are bound by
// dependent random gathers (queue -> row_ptr -> col -> C[u] -> Sigma_tot[c]).
// Each warp therefore works on several independent vertices at once (U-way
// interleave in the sub-warp kernel, E-way batched row loads elsewhere), and
// every queue append / counter update is aggregated per block so that no
// global address sees more than one atomic per block and tile.
#pragma once
#include "common.cuh"

// ---------------------------------------------------------------------------
// block-level helpers
// ---------------------------------------------------------------------------
template <int BT>
__device__ __forceinline__ ull block_sum_ull(ull x) {   // result valid in thread 0
    __shared__ ull sh[BT / 32];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(FULLMASK, x, o);
    __syncthreads();
    if (lane_id() == 0) sh[threadIdx.x >> 5] = x;
    __syncthreads();
    if (threadIdx.x == 0)
        for (int i = 1; i < BT / 32; ++i) x += sh[i];
    return x;
}

// K per-thread counters summed over the block and added to K global counters
// with one barrier (instead of one block reduction per counter)
template <int BT, int K>
__device__ __forceinline__ void block_add_counters(const ull (&x)[K], ull* const (&dst)[K]) {
    __shared__ ull sh[BT / 32][K];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        ull y = x[k];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) y += __shfl_xor_sync(FULLMASK, y, o);
        if (lane == 0) sh[wib][k] = y;
    }
    __syncthreads();
    if (threadIdx.x < K) {
        ull t = 0;
#pragma unroll
        for (int w = 0; w < BT / 32; ++w) t += sh[w][threadIdx.x];
        if (t) atomicAdd(dst[threadIdx.x], t);
    }
}

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
            if (sv) maxdeg[3] = 1;   // some self-loop: the level's s(v) are not all zero
            if ((ull)(e - b) > mymax) mymax = (ull)(e - b);
        }
    }
    if (lane == 0 && mymax) atomicMax(maxdeg, mymax);
}

// a1: every vertex its own community
__global__ void k_level_init(int n, const int64_t* __restrict__ d, int32_t* __restrict__ C,
                             int64_t* __restrict__ Sig, int32_t* __restrict__ size, int64_t* __restrict__ dp,
                             int32_t* __restrict__ stamp, int2* __restrict__ cst, Carry* __restrict__ carry,
                             PruneState ps) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n;
         v += (long long)gridDim.x * blockDim.x) {
        C[v] = (int32_t)v;
        Sig[v] = d[v];
        size[v] = 1;
        dp[v] = 0;
        stamp[v] = -1;
        cst[v] = make_int2((int)v, -1);
        if (ps.rmflag) ps.rmflag[v] = -1;
        if (ps.smflag) { ps.smflag[v] = -1; ps.chg[v] = -1; }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) { carry->iter = 0; carry->converged = 0; carry->log_base = 0; }
}

__global__ void k_iter_begin(IterCounters* ctr) {
    ull* p = reinterpret_cast<ull*>(ctr);
    for (int i = threadIdx.x; i < (int)(sizeof(IterCounters) / sizeof(ull)); i += blockDim.x) p[i] = 0;
}

// ---------------------------------------------------------------------------
// a2: MG pruning frontier (Eq. 6/7) fused with degree binning.
//   inactive iff  qW (2 d'(v) - d(v)) + p (minSig - Sig[C[v]]) d(v) >= 0
// Tiles of PB_BT*PB_IPT vertices; per-bin offsets are aggregated in shared
// memory, one global atomic per bin per tile.  Bin choice never changes
// results (P7).
// ---------------------------------------------------------------------------
struct BinThresholds {
    int t[NBINS - 1];   // upper row-length bound of bins 0..NBINS-2; the last bin takes the rest
};
#define PB_BT 256
#define PB_IPT 4

#ifndef GALA_PRUNE_EAGER
#define GALA_PRUNE_EAGER 0   // 1: row bounds + community size loaded up front (A/B: slower, 0.63 -> 0.67 ms on lfr1m; profiles/r01j_ab_prune.txt)
#endif
#ifndef GALA_PRUNE_MINB
#define GALA_PRUNE_MINB 4   // <= 64 registers: one wave of 1024-vertex tiles (A/B: lfr1m 0.76 -> 0.64 ms)
#endif
template <typename ST>
__global__ void __launch_bounds__(PB_BT, GALA_PRUNE_MINB) k_prune_bin(int vlo, int n, const int64_t* __restrict__ rp,
                                                     const int64_t* __restrict__ d, const int64_t* __restrict__ dp,
                                                     const int32_t* __restrict__ C, const int64_t* __restrict__ Sig,
                                                     const int32_t* __restrict__ size, PruneState ps, ST qW, ST p,
                                                     const Carry* __restrict__ carry, IterCounters* __restrict__ ctr,
                                                     QRec* __restrict__ queues, long long qstride, BinThresholds th) {
    __shared__ unsigned s_cnt[NBINS];
    __shared__ ull s_base[NBINS];
    const long long minSig = carry->minSig;
    const int prev = carry->iter - 1;   // the previous iteration of this level (-1: none)
    ull my_active = 0, my_pruned = 0;
    ull my_deg[NBINS];
#pragma unroll
    for (int b = 0; b < NBINS; ++b) my_deg[b] = 0;
    const long long tile = (long long)PB_BT * PB_IPT;
    for (long long t0 = vlo + (long long)blockIdx.x * tile; t0 < n; t0 += (long long)gridDim.x * tile) {
        if (threadIdx.x < NBINS) s_cnt[threadIdx.x] = 0;
        int bin[PB_IPT];
        bool act[PB_IPT];
        long long dv[PB_IPT], dpv[PB_IPT];
        int cv[PB_IPT];
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) {
            long long v = t0 + (long long)j * PB_BT + threadIdx.x;
            bool ok = v < n;
            dv[j] = ok ? d[v] : 0;
            dpv[j] = ok ? dp[v] : 0;
            cv[j] = ok ? C[v] : 0;
        }
        long long sg[PB_IPT];
#if GALA_PRUNE_EAGER
        // row bounds and the community size loaded with the vertex state / Sigma_tot gather (one
        // dependent round fewer for queued vertices; the extra bytes are coalesced or L2 hits)
        long long rb[PB_IPT], re[PB_IPT];
        int szv[PB_IPT];
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) {
            long long v = t0 + (long long)j * PB_BT + threadIdx.x;
            rb[j] = v < n ? rp[v] : 0;
            re[j] = v < n ? rp[v + 1] : 0;
        }
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) {
            sg[j] = dv[j] > 0 ? Sig[cv[j]] : 0;
            szv[j] = dv[j] > 0 ? size[cv[j]] : 0;
        }
#else
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) sg[j] = dv[j] > 0 ? Sig[cv[j]] : 0;
#endif
        int deg[PB_IPT];
        long long beg[PB_IPT];
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) {
            long long v = t0 + (long long)j * PB_BT + threadIdx.x;
            bin[j] = -1;
            deg[j] = 0;
            beg[j] = 0;
            act[j] = false;
            if (dv[j] > 0) {
                bool active = true;
                if (ps.mode == 1 || ps.mode == 4) {
                    ST lhs = qW * (ST)(2 * dpv[j] - dv[j]) + p * (ST)(minSig - sg[j]) * (ST)dv[j];
                    active = lhs < (ST)0;
                }
                if (ps.mode == 2 && prev >= 0)   // SM: some community around v changed
                    active = ps.chg[cv[j]] == prev || ps.smflag[v] == prev;
                if ((ps.mode == 3 || ps.mode == 4) && prev >= 0 && ps.rmflag[v] != prev)
                    active = false;              // RM: no neighbour moved
                act[j] = active;
                if (active) { my_active++; } else { my_pruned++; }
                if (active || ps.instr) {
#if GALA_PRUNE_EAGER
                    beg[j] = rb[j];
                    long long dg = re[j] - rb[j];
#else
                    beg[j] = rp[v];
                    long long dg = rp[v + 1] - beg[j];
#endif
                    deg[j] = (int)(dg > INT_MAX ? INT_MAX : dg);
                    int b = NBINS - 1;
#pragma unroll
                    for (int k = NBINS - 2; k >= 0; --k)
                        if (deg[j] <= th.t[k]) b = k;
                    bin[j] = b;
                    my_deg[b] += (ull)deg[j];
                }
            }
        }
#if !GALA_PRUNE_EAGER
        int szv[PB_IPT];
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) szv[j] = bin[j] >= 0 ? size[cv[j]] : 0;
#endif
        bool anyq = false;
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) anyq |= bin[j] >= 0;
        if (!__syncthreads_or(anyq)) continue;   // nothing queued in this tile (also: s_cnt reset visible)
        unsigned off[PB_IPT];
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) {
            unsigned peers = __match_any_sync(FULLMASK, bin[j]);
            int leader = __ffs(peers) - 1;
            unsigned base = 0;
            if (bin[j] >= 0 && lane_id() == leader) base = atomicAdd(&s_cnt[bin[j]], (unsigned)__popc(peers));
            base = __shfl_sync(FULLMASK, base, leader);
            off[j] = base + __popc(peers & lanemask_lt());
        }
        __syncthreads();
        if (threadIdx.x < NBINS)
            s_base[threadIdx.x] = s_cnt[threadIdx.x] ? atomicAdd(&ctr->bin_count[threadIdx.x], (ull)s_cnt[threadIdx.x]) : 0;
        __syncthreads();
#pragma unroll
        for (int j = 0; j < PB_IPT; ++j) {
            if (bin[j] >= 0) {
                QRec q;
                q.v = (int)(t0 + (long long)j * PB_BT + threadIdx.x);
                q.deg = deg[j];
                q.beg = beg[j];
                q.cv = cv[j];
                q.szv = szv[j];
                q.dv = dv[j];
                q.sigv = sg[j];
                q.pad = act[j] ? 1 : 0;   // 0: queued only for the FN/FP instrumentation
                qview(queues, qstride, bin[j])[(long long)s_base[bin[j]] + off[j]] = q;
            }
        }
    }
    ull vals[NBINS + 2];
    ull* dsts[NBINS + 2];
#pragma unroll
    for (int b = 0; b < NBINS; ++b) { vals[b] = my_deg[b]; dsts[b] = &ctr->bin_deg[b]; }
    vals[NBINS] = my_active; dsts[NBINS] = &ctr->n_active;
    vals[NBINS + 1] = my_pruned; dsts[NBINS + 1] = &ctr->n_pruned;
    block_add_counters<PB_BT, NBINS + 2>(vals, dsts);
}

// ---------------------------------------------------------------------------
// a5: apply moves (Alg. 1 line 5) for every queued (active) vertex whose
// decision differs: Sigma_tot and sizes by int atomics (order-independent),
// C[v] <- nextC[v], stamp[v] <- iteration, and the moved list (v, old) with
// one global atomic per block and tile.
// ---------------------------------------------------------------------------
#define AP_BT 256
// Delta-update work items: a mover with at most DCH entries is one item, a
// longer one is split into ceil(deg/DCH) chunk items so a hub's row is spread
// over many warps instead of serialising one (its d' is then summed by
// atomics onto a zero written here).  Item capacity: n + nnz/DCH.
#define DCH 256
#define DLIGHT 64   // movers with rows up to this many entries: half-warp delta items
__global__ void __launch_bounds__(AP_BT) k_apply(IterCounters* __restrict__ ctr, QRec* queues,
                                                 long long qstride, const int32_t* __restrict__ nextC,
                                                 int32_t* __restrict__ C, int64_t* __restrict__ Sig,
                                                 int32_t* __restrict__ size, int64_t* __restrict__ dp,
                                                 int32_t* __restrict__ stamp, int2* __restrict__ cst,
                                                 const Carry* __restrict__ carry, int32_t* __restrict__ it_v, int32_t* __restrict__ it_old,
                                                 int32_t* __restrict__ it_chunk, PruneState ps, long long icap,
                                                 int agg32) {
    __shared__ unsigned s_cnt, s_items, s_hitems;
    __shared__ unsigned s_scr[AP_BT / 32][32];
    __shared__ ull s_ibase, s_hbase;
    long long cnt[NBINS];
    long long total = 0;
#pragma unroll
    for (int b = 0; b < NBINS; ++b) { cnt[b] = (long long)ctr->bin_count[b]; total += cnt[b]; }
    if ((long long)blockIdx.x * AP_BT >= total) return;   // no queued vertex for this block
    const int iter_id = carry->iter;
    const int lane = lane_id();
    ull my_deg = 0, my_fn = 0, my_fp = 0;
    for (long long t0 = (long long)blockIdx.x * AP_BT; t0 < total; t0 += (long long)gridDim.x * AP_BT) {
        long long i = t0 + threadIdx.x;
        bool mover = false;
        int v = 0, oc = 0, deg = 0, mnc = 0;
        unsigned mdv = 0;
        if (i < total) {
            int b = 0;
            long long r = i;
#pragma unroll
            for (int k = 0; k < NBINS - 1; ++k)
                if (b == k && r >= cnt[k]) { r -= cnt[k]; b = k + 1; }
            const QRec q = qview(queues, qstride, b)[r];
            v = q.v;
            int nc = nextC[v];
            oc = q.cv;
            if (ps.instr) {
                if (!q.pad) { my_fn += nc != oc; nc = oc; }   // pruned: would it have moved?  it stays
                else my_fp += nc == oc;
            }
            if (nc != oc) {
                mover = true;
                if (ps.chg) { ps.chg[oc] = iter_id; ps.chg[nc] = iter_id; }
                long long dv = q.dv;
                deg = q.deg;
                C[v] = nc;
                stamp[v] = iter_id;
                cst[v] = make_int2(nc, iter_id);
                if (!agg32) {
                    atomicAdd(reinterpret_cast<ull*>(&Sig[oc]), (ull)(-dv));
                    atomicAdd(reinterpret_cast<ull*>(&Sig[nc]), (ull)dv);
                    atomicSub(&size[oc], 1);
                    atomicAdd(&size[nc], 1);
                }
                my_deg += (ull)q.deg;
                if (deg > DCH) dp[v] = 0;   // chunk items add onto it
                mdv = (unsigned)dv;
                mnc = nc;
            }
        }
        if (agg32) {   // d(v) < 2^32: the warp's movers into / out of the same community are combined
                       // (match_any + a shared group sum) into one Sigma_tot and one size atomic
            const unsigned pn = __match_any_sync(FULLMASK, mover ? mnc : -1 - lane);
            const unsigned sn = group_sum(pn, mover ? mdv : 0u, s_scr[threadIdx.x >> 5]);
            if (mover && lane == __ffs(pn) - 1) {
                atomicAdd(reinterpret_cast<ull*>(&Sig[mnc]), (ull)sn);
                atomicAdd(&size[mnc], __popc(pn));
            }
            const unsigned po = __match_any_sync(FULLMASK, mover ? oc : -1 - lane);
            const unsigned so = group_sum(po, mover ? mdv : 0u, s_scr[threadIdx.x >> 5]);
            if (mover && lane == __ffs(po) - 1) {
                atomicAdd(reinterpret_cast<ull*>(&Sig[oc]), (ull)(-(long long)so));
                atomicSub(&size[oc], __popc(po));
            }
        }
        // items of this thread: a light mover (row <= DLIGHT) is one item at the FRONT of the
        // item arrays (half-warp per item in k_dp_delta), any other mover is one item or the chunk
        // count of a heavy mover at the BACK (warp per item)
        const bool light = mover && deg <= DLIGHT;
        const unsigned nit = (!mover || light) ? 0u : (deg > DCH ? (unsigned)((deg + DCH - 1) / DCH) : 1u);
        unsigned incl = nit;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned y = __shfl_up_sync(FULLMASK, incl, o);
            if (lane >= o) incl += y;
        }
        if (threadIdx.x == 0) { s_cnt = 0; s_items = 0; s_hitems = 0; }
        __syncthreads();
        const unsigned m = __ballot_sync(FULLMASK, mover);
        if (m && lane == 0) atomicAdd(&s_cnt, (unsigned)__popc(m));
        const unsigned lm = __ballot_sync(FULLMASK, light);
        unsigned loff = 0;
        if (lm && lane == 0) loff = atomicAdd(&s_items, (unsigned)__popc(lm));
        loff = __shfl_sync(FULLMASK, loff, 0) + __popc(lm & lanemask_lt());
        unsigned ioff = 0;
        const unsigned wtot = __shfl_sync(FULLMASK, incl, 31);
        if (lane == 31 && wtot) ioff = atomicAdd(&s_hitems, wtot);
        ioff = __shfl_sync(FULLMASK, ioff, 31) + incl - nit;
        __syncthreads();
        if (threadIdx.x == 0) {
            if (s_cnt) atomicAdd(&ctr->n_moved, (ull)s_cnt);
            s_ibase = s_items ? atomicAdd(&ctr->n_items, (ull)s_items) : 0;
            s_hbase = s_hitems ? atomicAdd(&ctr->n_items_hi, (ull)s_hitems) : 0;
        }
        __syncthreads();
        if (light) {
            const ull at = s_ibase + loff;
            it_v[at] = v;
            it_old[at] = oc;
            it_chunk[at] = 0;
        }
        for (unsigned j = 0; j < nit; ++j) {
            const long long at = icap - 1 - (long long)(s_hbase + ioff + j);
            it_v[at] = v;
            it_old[at] = oc;
            it_chunk[at] = (int32_t)j;
        }
        __syncthreads();   // s_ibase reused by the next tile
    }
    ull md = block_sum_ull<AP_BT>(my_deg);
    if (threadIdx.x == 0 && md) atomicAdd(&ctr->moved_deg, md);
    if (ps.instr) {
        ull f = block_sum_ull<AP_BT>(my_fn);
        if (threadIdx.x == 0 && f) atomicAdd(&ctr->n_fn, f);
        f = block_sum_ull<AP_BT>(my_fp);
        if (threadIdx.x == 0 && f) atomicAdd(&ctr->n_fp, f);
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
                                                  const int32_t* __restrict__ C, const int2* __restrict__ cst,
                                                  const int32_t* __restrict__ it_v, const int32_t* __restrict__ it_old,
                                                  const int32_t* __restrict__ it_chunk,
                                                  const int32_t* __restrict__ stamp, int64_t* __restrict__ dp,
                                                  const Carry* __restrict__ carry, long long nnz, int mode,
                                                  long long fnum, long long fden, int32_t* __restrict__ ckey,
                                                  const int32_t* __restrict__ rev, int32_t* __restrict__ rmflag,
                                                  int n, long long icap) {
    if (!use_delta(ctr, nnz, mode, fnum, fden)) {   // full recompute follows: clear d' (k_dp_zero fused)
        for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n;
             v += (long long)gridDim.x * blockDim.x)
            dp[v] = 0;
        return;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        ctr->delta_used = 1;
        if (ckey) const_cast<Carry*>(carry)->ckey_valid = 0;   // per-entry communities now stale
    }
    (void)rev;
    const int iter_id = carry->iter;
    const int lane = lane_id();
    long long wid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    // light movers (rows <= DLIGHT = 64): a half-warp per item, 4 entries per lane, two items per warp
    {
        const long long ml = (long long)ctr->n_items;
        const int hl = lane & 15, half = lane >> 4;
        for (long long i0 = wid * 2; i0 < ml; i0 += nw * 2) {   // warp-uniform
            const long long i = i0 + half;
            const bool ok = i < ml;
            const int u = ok ? it_v[i] : 0, oc = ok ? it_old[i] : -1;
            const int nc = ok ? C[u] : -1;
            const int64_t b = ok ? rp[u] : 0, e = ok ? rp[u + 1] : 0;
            int x[4], cx[4], sx[4];
            long long wt[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int64_t j = b + hl + 16 * t;
                x[t] = j < e ? col[j] : u;
                wt[t] = (UNIT || j >= e) ? 1 : w[j];
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int2 cs = x[t] != u ? cst[x[t]] : make_int2(-1, iter_id);   // one 8-byte gather
                cx[t] = cs.x;
                sx[t] = cs.y;
            }
            long long acc = 0;
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (x[t] == u) continue;
                if (rmflag) rmflag[x[t]] = iter_id;
                if (cx[t] == nc) acc += wt[t];
                if (sx[t] != iter_id) {
                    if (cx[t] == oc) atomicAdd(reinterpret_cast<ull*>(&dp[x[t]]), (ull)(-wt[t]));
                    else if (cx[t] == nc) atomicAdd(reinterpret_cast<ull*>(&dp[x[t]]), (ull)wt[t]);
                }
            }
#pragma unroll
            for (int o = 8; o > 0; o >>= 1) acc += __shfl_xor_sync(FULLMASK, acc, o);
            if (ok && hl == 0) dp[u] = acc;
        }
    }
    const long long m = (long long)ctr->n_items_hi;
    for (long long i = wid; i < m; i += nw) {
        const long long ii = icap - 1 - i;
        const int u = it_v[ii], oc = it_old[ii], ch = it_chunk[ii];
        const int nc = C[u];
        const int64_t rb = rp[u], re = rp[u + 1];
        const bool heavy = re - rb > DCH;
        const int64_t b = rb + (int64_t)ch * DCH, e = heavy ? min(b + DCH, re) : re;
        long long acc = 0;
        for (int64_t j0 = b; j0 < e; j0 += 128) {   // 4 entries per lane in flight
            int x[4], cx[4], sx[4];
            long long wt[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int64_t j = j0 + lane + 32 * t;
                x[t] = j < e ? col[j] : u;
                wt[t] = (UNIT || j >= e) ? 1 : w[j];
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int2 cs = x[t] != u ? cst[x[t]] : make_int2(-1, iter_id);
                cx[t] = cs.x;
                sx[t] = cs.y;
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (x[t] == u) continue;
                if (rmflag) rmflag[x[t]] = iter_id;   // RM: a neighbour of x moved
                if (cx[t] == nc) acc += wt[t];
                if (sx[t] != iter_id) {
                    if (cx[t] == oc) atomicAdd(reinterpret_cast<ull*>(&dp[x[t]]), (ull)(-wt[t]));
                    else if (cx[t] == nc) atomicAdd(reinterpret_cast<ull*>(&dp[x[t]]), (ull)wt[t]);
                }
            }
        }
        acc = warp_sum_ll(acc);
        if (lane == 0) {
            if (heavy) { if (acc) atomicAdd(reinterpret_cast<ull*>(&dp[u]), (ull)acc); }
            else dp[u] = acc;
        }
    }
}

// d'(v) = sum of w(v,u), u != v, C[u] == C[v]   (definition), edge-parallel:
// every lane takes entries (row r, col u) 32 apart (4 in flight), equal rows of
// a 32-entry chunk are summed with __match_any_sync and one atomic per row.
__global__ void k_dp_zero(IterCounters* __restrict__ ctr, int vlo, int vhi, int64_t* __restrict__ dp, long long nnz,
                          int mode, long long fnum, long long fden) {
    if (use_delta(ctr, nnz, mode, fnum, fden)) return;
    for (long long v = vlo + (long long)blockIdx.x * blockDim.x + threadIdx.x; v < vhi;
         v += (long long)gridDim.x * blockDim.x)
        dp[v] = 0;
}

template <bool UNIT>
__global__ void __launch_bounds__(256) k_dp_full(IterCounters* __restrict__ ctr, long long nnz,
                                                 const int32_t* __restrict__ row, const int32_t* __restrict__ col,
                                                 const int64_t* __restrict__ w, const int32_t* __restrict__ C,
                                                 int64_t* __restrict__ dp, int mode, long long fnum, long long fden,
                                                 int32_t* __restrict__ ckey, int* __restrict__ carry_valid,
                                                 int32_t* __restrict__ rmflag, const int32_t* __restrict__ stamp,
                                                 const Carry* __restrict__ carry) {
    if (use_delta(ctr, nnz, mode, fnum, fden)) return;
    const int iter_id = rmflag ? carry->iter : 0;
    if (ckey && blockIdx.x == 0 && threadIdx.x == 0) carry_valid[0] = 1;   // rewritten below for every entry
    const int lane = lane_id();
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long base = (((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 128; base < nnz;
         base += nw * 128) {
        int r[4], u[4];
        long long wt[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            long long e = base + lane + 32 * t;
            r[t] = e < nnz ? row[e] : -1;
            u[t] = e < nnz ? col[e] : -1;
            wt[t] = (e < nnz && !UNIT) ? w[e] : 1;
        }
        int cr[4], cu[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            cr[t] = r[t] >= 0 ? C[r[t]] : 0;
            cu[t] = u[t] >= 0 ? C[u[t]] : 1;
        }
        if (rmflag) {   // RM: mark rows with a neighbour that moved in this iteration
#pragma unroll
            for (int t = 0; t < 4; ++t)
                if (r[t] >= 0 && u[t] != r[t] && stamp[u[t]] == iter_id) rmflag[r[t]] = iter_id;
        }
        if (ckey) {   // refresh the per-entry neighbour communities for the next decide
#pragma unroll
            for (int t = 0; t < 4; ++t)
                if (r[t] >= 0) ckey[base + lane + 32 * t] = u[t] == r[t] ? -1 : cu[t];
        }
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const bool hit = r[t] >= 0 && u[t] != r[t] && cu[t] == cr[t];
            const unsigned peers = __match_any_sync(FULLMASK, r[t]);
            ull sum;
            if (UNIT) {
                sum = (ull)__popc(__ballot_sync(FULLMASK, hit) & peers);
            } else {   // rows are contiguous lane runs: segmented tree sum, leader = first lane of the run
                long long x = hit ? wt[t] : 0;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const long long y = __shfl_down_sync(FULLMASK, x, o);
                    const int ro = __shfl_down_sync(FULLMASK, r[t], o);
                    if (lane + o < 32 && ro == r[t]) x += y;
                }
                sum = (ull)x;
            }
            if (r[t] >= 0 && lane == __ffs(peers) - 1 && sum) atomicAdd(reinterpret_cast<ull*>(&dp[r[t]]), sum);
        }
    }
}

// ---------------------------------------------------------------------------
// a7: sumDC = sum_v (d'(v) + s(v)), S2 = sum_c Sig[c]^2 (int128), minSig =
// min{Sig > 0} (Alg. 1 lines 8-11).  N' = qW sumDC - p S2.  The last block
// to finish combines the per-block partials and takes the convergence
// decision dN < T (Alg. 1 lines 12-13) on the device.
// mode 0: level start (N := N'), mode 1: iteration end.
// SM pruning history: entry (r, u) marks row r when the community of
// u gained or lost a member in this iteration (communities after the moves).
// Edge-parallel over all entries; only launched with the SM strategy.
__global__ void __launch_bounds__(256) k_sm_flags(long long nnz, const int32_t* __restrict__ row,
                                                  const int32_t* __restrict__ col, const int32_t* __restrict__ C,
                                                  PruneState ps, const Carry* __restrict__ carry) {
    const int iter_id = carry->iter;
    for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x; e < nnz;
         e += (long long)gridDim.x * blockDim.x) {
        const int u = col[e];
        if (ps.chg[C[u]] == iter_id) ps.smflag[row[e]] = iter_id;
    }
}

// end-of-iteration bookkeeping shared by k_record and the fused k_reduce: append
// the counters to the device log, advance the iteration index and (graph mode)
// set the loop condition of the enclosing conditional while-node: continue iff
// not converged, under the iteration cap and with room in the log.
__device__ __forceinline__ void record_iteration(const IterCounters* ctr, Carry* carry, IterLog* log, int log_cap,
                                                 int max_iters, unsigned long long cond_handle) {
    const int it = carry->iter;
    const int slot = it - carry->log_base;
    if (slot >= 0 && slot < log_cap) {
        IterLog& L = log[slot];
        L.ctr = *ctr;
        L.N_hi = carry->N_hi;
        L.N_lo = carry->N_lo;
        L.converged = carry->converged;
        L.t_ns = carry->t_ns;
    }
    carry->iter = it + 1;
    const int more = !carry->converged && (max_iters <= 0 || it + 1 < max_iters) && (slot + 1 < log_cap);
    carry->more = more;
    if (cond_handle) cudaGraphSetConditional((cudaGraphConditionalHandle)cond_handle, more ? 1u : 0u);
}

// ---------------------------------------------------------------------------
#ifndef GALA_REDUCE_PTAIL
#define GALA_REDUCE_PTAIL 1   // last block copies / clears the iteration counters with all its threads
#endif
#ifndef GALA_REDUCE_U
#define GALA_REDUCE_U 4   // (<= 64 registers: 4 blocks per SM) Sigma_tot / d' values per thread per batch in k_reduce (0: the strided loops)
#endif
template <int BT>
__global__ void __launch_bounds__(BT) k_reduce(int n, int dlo, int dhi, const int64_t* __restrict__ dp,
                                               const int64_t* __restrict__ s, const int64_t* __restrict__ Sig,
                                               long long* __restrict__ part_dc, i128* __restrict__ part_s2,
                                               long long* __restrict__ part_min, IterCounters* __restrict__ ctr,
                                               Carry* __restrict__ carry, long long qW_hi, ull qW_lo, long long p,
                                               long long T_hi, ull T_lo, int mode, IterLog* __restrict__ log = nullptr,
                                               int log_cap = 0, int max_iters = 0,
                                               unsigned long long cond_handle = 0) {
    __shared__ long long sh_dc[BT / 32];
    __shared__ i128 sh_s2[BT / 32];
    __shared__ long long sh_min[BT / 32];
    __shared__ bool amLast;
    __shared__ int s_tail, s_slot;
    long long dc = 0, mn = LLONG_MAX;
    i128 s2 = 0;
    const long long stride = (long long)gridDim.x * BT;
#if GALA_REDUCE_U > 0
    // every load of a batch (U Sigma_tot and U d' (+ s) values per thread) issued before any use:
    // one memory latency per batch instead of one per tail element (latency-bound kernel)
    for (long long v0 = (long long)blockIdx.x * BT + threadIdx.x; v0 < n; v0 += GALA_REDUCE_U * stride) {
        long long g[GALA_REDUCE_U], q[GALA_REDUCE_U], r[GALA_REDUCE_U];
#pragma unroll
        for (int k = 0; k < GALA_REDUCE_U; ++k) {
            const long long v = v0 + k * stride, x = dlo + v;
            g[k] = v < n ? Sig[v] : 0;
            q[k] = x < dhi ? dp[x] : 0;
            r[k] = (s && x < dhi) ? s[x] : 0;
        }
#pragma unroll
        for (int k = 0; k < GALA_REDUCE_U; ++k) {
            s2 += (i128)g[k] * g[k];
            if (g[k] > 0 && g[k] < mn) mn = g[k];
            dc += q[k] + r[k];
        }
    }
#else
    long long v = (long long)blockIdx.x * BT + threadIdx.x;
    for (; v + 3 * stride < n; v += 4 * stride) {
        long long g0 = Sig[v], g1 = Sig[v + stride], g2 = Sig[v + 2 * stride], g3 = Sig[v + 3 * stride];
        s2 += (i128)g0 * g0 + (i128)g1 * g1 + (i128)g2 * g2 + (i128)g3 * g3;
        if (g0 > 0 && g0 < mn) mn = g0;
        if (g1 > 0 && g1 < mn) mn = g1;
        if (g2 > 0 && g2 < mn) mn = g2;
        if (g3 > 0 && g3 < mn) mn = g3;
    }
    for (; v < n; v += stride) {
        long long sg = Sig[v];
        s2 += (i128)sg * sg;
        if (sg > 0 && sg < mn) mn = sg;
    }
    v = dlo + (long long)blockIdx.x * BT + threadIdx.x;
    if (s) {
        for (; v + 3 * stride < dhi; v += 4 * stride)
            dc += dp[v] + dp[v + stride] + dp[v + 2 * stride] + dp[v + 3 * stride] + s[v] + s[v + stride] +
                  s[v + 2 * stride] + s[v + 3 * stride];
        for (; v < dhi; v += stride) dc += dp[v] + s[v];
    } else {   // level without self-loops (s == 0): only d'
        for (; v + 3 * stride < dhi; v += 4 * stride)
            dc += dp[v] + dp[v + stride] + dp[v + 2 * stride] + dp[v + 3 * stride];
        for (; v < dhi; v += stride) dc += dp[v];
    }
#endif
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
    if (!amLast) return;
    // last block: combine the per-block partials in parallel
    __threadfence();
    long long tdc = 0, tmn = LLONG_MAX;
    i128 ts2 = 0;
    for (int b = threadIdx.x; b < (int)gridDim.x; b += BT) {
        tdc += *(volatile long long*)&part_dc[b];
        ts2 += mk128(*(volatile long long*)((volatile char*)&part_s2[b] + 8), *(volatile ull*)&part_s2[b]);
        long long m2 = *(volatile long long*)&part_min[b];
        tmn = m2 < tmn ? m2 : tmn;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        tdc += __shfl_xor_sync(FULLMASK, tdc, o);
        ts2 += shfl_xor_st(ts2, o);
        long long om = __shfl_xor_sync(FULLMASK, tmn, o);
        tmn = om < tmn ? om : tmn;
    }
    __syncthreads();
    if (lane == 0) { sh_dc[wib] = tdc; sh_s2[wib] = ts2; sh_min[wib] = tmn; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < BT / 32; ++i) {
            tdc += sh_dc[i];
            ts2 += sh_s2[i];
            tmn = sh_min[i] < tmn ? sh_min[i] : tmn;
        }
        carry->S2_hi = hi128(ts2);
        carry->S2_lo = lo128(ts2);
        carry->minSig = tmn;
        carry->sumDC = tdc;
        carry->t_ns = globaltimer_ns();
        s_tail = 0;
        if (mode & 2) {   // multi-GPU: sumDC is rank-local; k_finish completes after the all-reduce
            ctr->ticket = 0;
        } else {
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
        if (log) {   // k_record fused: log the iteration, advance, set the loop condition, clear counters
#if GALA_REDUCE_PTAIL
            // the counter copy into the log and the clear are done by the whole block below
            const int it = carry->iter;
            const int slot = it - carry->log_base;
            s_slot = (slot >= 0 && slot < log_cap) ? slot : -1;
            if (s_slot >= 0) {
                IterLog& L = log[slot];
                L.N_hi = carry->N_hi;
                L.N_lo = carry->N_lo;
                L.converged = carry->converged;
                L.t_ns = carry->t_ns;
            }
            carry->iter = it + 1;
            const int more = !carry->converged && (max_iters <= 0 || it + 1 < max_iters) && (slot + 1 < log_cap);
            carry->more = more;
            if (cond_handle) cudaGraphSetConditional((cudaGraphConditionalHandle)cond_handle, more ? 1u : 0u);
            s_tail = 1;
#else
            record_iteration(ctr, carry, log, log_cap, max_iters, cond_handle);
            ull* c = reinterpret_cast<ull*>(ctr);
            for (int i = 0; i < (int)(sizeof(IterCounters) / sizeof(ull)); ++i) c[i] = 0;
#endif
        }
        }   // mode & 2
    }
#if GALA_REDUCE_PTAIL
    __syncthreads();
    if (s_tail) {   // log[slot].ctr = *ctr; *ctr = 0 -- one counter per thread (same values as record_iteration)
        ull* c = reinterpret_cast<ull*>(ctr);
        for (int i = threadIdx.x; i < (int)(sizeof(IterCounters) / sizeof(ull)); i += BT) {
            const ull x = c[i];
            if (s_slot >= 0) reinterpret_cast<ull*>(&log[s_slot].ctr)[i] = x;
            c[i] = 0;
        }
    }
#endif
}

// ---------------------------------------------------------------------------
// end of iteration: append the counters to the device log, advance the
// iteration index and (graph mode) set the loop condition of the enclosing
// conditional while-node: continue iff not converged, under the iteration
// cap and with room in the log.
// ---------------------------------------------------------------------------
__global__ void k_record(const IterCounters* __restrict__ ctr, Carry* __restrict__ carry, IterLog* __restrict__ log,
                         int log_cap, int max_iters, unsigned long long cond_handle) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    record_iteration(ctr, carry, log, log_cap, max_iters, cond_handle);
}

// level-0 init of the per-entry neighbour communities: C = identity
__global__ void k_ckey_init(long long nnz, const int32_t* __restrict__ row, const int32_t* __restrict__ col,
                            int32_t* __restrict__ ckey, Carry* __restrict__ carry) {
    if (blockIdx.x == 0 && threadIdx.x == 0) carry->ckey_valid = 1;
    for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (long long)gridDim.x * blockDim.x)
        ckey[e] = col[e] == row[e] ? -1 : col[e];
}

