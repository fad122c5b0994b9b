// fabric.cuh — device-resident multi-GPU iteration over peer memory (§4.3, P:318-324;
// SURVEY.md §8(a) a10, §8(e), §8(f) NEXT #1).
//
// One process per GPU; every rank maps a small symmetric region of every other rank
// (CUDA IPC over NVLink / NVSwitch, or plain pointers when the "ranks" are threads of one
// process on one device -- the loopback test backend).  A phase-1 iteration then runs
// entirely on the device, with no host round trip, and is captured into the level's
// conditional CUDA graph exactly like the single-GPU one:
//
//   prune + decide over the owned rows            (the single-GPU kernels)
//   k_collect_moves                               owned movers -> (v, new) list
//   k_fab_push (+ k_fab_push_fix)                 the list, or this rank's label slice,
//                                                 stored into EVERY rank's inbox slot
//                                                 (P2P stores); per-sender choice:
//                                                 sparse iff 8 m_r < 4 n_r
//   k_fab_barrier                                 all slots written
//   k_fab_apply                                   every rank applies every slot to its
//                                                 replica (C, Sigma_tot, size, stamp; int
//                                                 atomics, order-independent -> replicas
//                                                 stay bit-identical), builds the d' items
//   k_fab_dp_delta | k_dp_zero + k_dp_full        §3.5 delta update across ranks: a moved
//                                                 vertex u pushes +-w along its MIRROR row
//                                                 (the owned neighbours of u), owned movers
//                                                 recompute from their own row; full
//                                                 recompute of the owned rows when the
//                                                 moved volume is large
//   k_reduce (rank-local sum d'+s; S2, min over the replicated Sigma_tot)
//   k_fab_scal                                    per-rank scalars into every rank's slot
//   k_fab_barrier                                 all scalars written
//   k_fab_finish                                  sum in rank order, N, convergence (ΔN < T),
//                                                 device log, loop condition
//
// Inbox and scalar slots are double-buffered by iteration parity: a sender can be at most
// one iteration ahead of a receiver (it must pass the receiver's barrier arrival of that
// iteration), so the parity it writes is never the one being read.
#pragma once
#include "common.cuh"

#define FAB_MAXP 16
#define FAB_NSCAL 8
#define FAB_SPARSE 1ull
#define FAB_DENSE 2ull

struct FabDev {
    int P, rank;
    ull* arrive[FAB_MAXP];       // barrier arrival counter of every rank
    int32_t* inbox[FAB_MAXP];    // inbox of every rank: 2 parities x istride ints
    ull* hdr[FAB_MAXP];          // per rank: 2 parities x FAB_MAXP headers (mode << 62 | count)
    long long* scal[FAB_MAXP];   // per rank: 2 parities x FAB_MAXP x FAB_NSCAL
    ull* epoch;                  // this rank: barriers passed so far
    int* err;                    // this rank: a barrier timed out (a peer died)
    long long istride;           // ints per inbox parity
    long long bnd[FAB_MAXP + 1]; // owned vertex ranges of this level
    long long off[FAB_MAXP];     // slot start (ints, even) of every sender in an inbox parity
    int force_dense;             // option sync_mode = 1: every sender exchanges its whole slice
    ull timeout_ns;              // barrier wait before giving up (env GALA_FABRIC_TIMEOUT_MS, default 20 s)
    ull* diag;                   // this rank: [epoch, counter seen] of the barrier that timed out
};

__device__ __forceinline__ ull ld_acquire_sys(const ull* p) {
    ull v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// All ranks arrive (one system-scope atomic on every peer's counter), then wait until this
// rank's counter shows P arrivals for this barrier.  A barrier that waits longer than the
// timeout (a peer died) sets the error flag and lets the run finish instead of hanging the GPU.
__global__ void k_fab_barrier(FabDev f) {
    const int lane = threadIdx.x;
    __threadfence_system();
    if (lane < f.P) atomicAdd_system(f.arrive[lane], 1ull);
    if (lane == 0) {
        const ull target = (*f.epoch + 1) * (ull)f.P;
        const ull t0 = globaltimer_ns();
        ull seen;
        while ((seen = ld_acquire_sys(f.arrive[f.rank])) < target) {
            if (globaltimer_ns() - t0 > f.timeout_ns) {
                if (!*f.err) { f.diag[0] = *f.epoch; f.diag[1] = seen; }
                *f.err = 1;
                break;
            }
            __nanosleep(64);
        }
        *f.epoch += 1;
        __threadfence_system();
    }
}

__device__ __forceinline__ int fab_par(const Carry* carry) { return carry->iter & 1; }

// this rank's movers (or its whole label slice) into every rank's inbox slot `rank`
__global__ void __launch_bounds__(256) k_fab_push(FabDev f, const int2* __restrict__ lmoves, const ull* __restrict__ lcount,
                                                  const int32_t* __restrict__ C, const Carry* __restrict__ carry) {
    const int par = fab_par(carry);
    const long long m = (long long)*lcount;
    const long long b = f.bnd[f.rank], ns = f.bnd[f.rank + 1] - b;
    const bool sparse = !f.force_dense && 2 * m < ns;   // 8 bytes per move vs 4 bytes per owned label
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x, nth = (long long)gridDim.x * blockDim.x;
    if (tid < f.P)
        f.hdr[tid][par * FAB_MAXP + f.rank] = ((sparse ? FAB_SPARSE : FAB_DENSE) << 62) | (ull)m;
    for (int p = 0; p < f.P; ++p) {
        int32_t* slot = f.inbox[p] + (long long)par * f.istride + f.off[f.rank];
        if (sparse) {
            int2* s2 = reinterpret_cast<int2*>(slot);
            for (long long i = tid; i < m; i += nth) s2[i] = lmoves[i];
        } else {
            for (long long i = tid; i < ns / 2; i += nth) {   // slot start is even: 8-byte stores
                const int2 x = make_int2(C[b + 2 * i], C[b + 2 * i + 1]);
                reinterpret_cast<int2*>(slot)[i] = x;
            }
            if ((ns & 1) && tid == 0) slot[ns - 1] = C[b + ns - 1];
        }
    }
    __threadfence_system();
}

// dense senders: the movers overwrite their labels in the slices just stored (stream order)
__global__ void k_fab_push_fix(FabDev f, const int2* __restrict__ lmoves, const ull* __restrict__ lcount,
                               const Carry* __restrict__ carry) {
    const int par = fab_par(carry);
    const long long m = (long long)*lcount;
    const long long b = f.bnd[f.rank], ns = f.bnd[f.rank + 1] - b;
    if (!f.force_dense && 2 * m < ns) return;
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x, nth = (long long)gridDim.x * blockDim.x;
    for (int p = 0; p < f.P; ++p) {
        int32_t* slot = f.inbox[p] + (long long)par * f.istride + f.off[f.rank];
        for (long long i = tid; i < m; i += nth) slot[lmoves[i].x - b] = lmoves[i].y;
    }
    __threadfence_system();
}

// Every slot of this rank's inbox applied to the replica: sparse slots list (v, new), dense
// slots hold the sender's whole label slice (a vertex moved iff its label differs).  The d'
// work items are built as in k_apply: one per mover with <= DCH row entries, else one per
// DCH-entry chunk; the row of an owned mover is its own row (recompute + push), the row of a
// remote mover is its mirror row (push only; no owned neighbour -> no item).
__global__ void __launch_bounds__(256) k_fab_apply(FabDev f, const Carry* __restrict__ carry, IterCounters* __restrict__ ctr,
                                                   int32_t* __restrict__ C, int64_t* __restrict__ Sig,
                                                   int32_t* __restrict__ size, const int64_t* __restrict__ d,
                                                   int32_t* __restrict__ stamp, int64_t* __restrict__ dp,
                                                   const int64_t* __restrict__ rp, const int64_t* __restrict__ mrp,
                                                   long long lv0, long long lv1, int32_t* __restrict__ it_v,
                                                   int32_t* __restrict__ it_old, int32_t* __restrict__ it_chunk) {
    __shared__ long long s_pre[FAB_MAXP + 1];
    __shared__ int s_sparse[FAB_MAXP];
    __shared__ unsigned s_cnt, s_items;
    __shared__ ull s_ibase;
    const int par = fab_par(carry);
    const int iter_id = carry->iter;
    const int32_t* ib = f.inbox[f.rank] + (long long)par * f.istride;
    const ull* hd = f.hdr[f.rank] + par * FAB_MAXP;
    if (threadIdx.x == 0) {
        long long acc = 0;
        for (int s = 0; s < f.P; ++s) {
            const ull h = hd[s];
            const bool sp = (h >> 62) == FAB_SPARSE;
            s_sparse[s] = sp;
            s_pre[s] = acc;
            acc += sp ? (long long)(h & ((1ull << 62) - 1)) : f.bnd[s + 1] - f.bnd[s];
        }
        s_pre[f.P] = acc;
        if (blockIdx.x == 0) {   // exchange statistics (trace / bench): dense senders, bytes received
            ull nd = 0, xb = 0;
            for (int s = 0; s < f.P; ++s) {
                nd += s_sparse[s] ? 0 : 1;
                xb += s_sparse[s] ? 8ull * (hd[s] & ((1ull << 62) - 1)) : 4ull * (ull)(f.bnd[s + 1] - f.bnd[s]);
            }
            ctr->n_dense = nd;
            ctr->xbytes = xb;
        }
    }
    __syncthreads();
    const long long total = s_pre[f.P];
    const int lane = lane_id();
    ull my_deg = 0;
    for (long long t0 = (long long)blockIdx.x * blockDim.x; t0 < total; t0 += (long long)gridDim.x * blockDim.x) {
        const long long i = t0 + threadIdx.x;
        bool mover = false;
        int v = 0, oc = 0;
        long long len = 0;
        if (i < total) {
            int s = 0;
            while (s + 1 < f.P && i >= s_pre[s + 1]) ++s;
            const long long j = i - s_pre[s];
            int nc;
            if (s_sparse[s]) {
                const int2 x = reinterpret_cast<const int2*>(ib + f.off[s])[j];
                v = x.x;
                nc = x.y;
            } else {
                v = (int)(f.bnd[s] + j);
                nc = ib[f.off[s] + j];
            }
            oc = C[v];
            if (nc != oc) {
                mover = true;
                const long long dv = d[v];
                C[v] = nc;
                stamp[v] = iter_id;
                atomicAdd(reinterpret_cast<ull*>(&Sig[oc]), (ull)(-dv));
                atomicAdd(reinterpret_cast<ull*>(&Sig[nc]), (ull)dv);
                atomicSub(&size[oc], 1);
                atomicAdd(&size[nc], 1);
                const bool own = v >= lv0 && v < lv1;
                len = own ? rp[v + 1] - rp[v] : mrp[v + 1] - mrp[v];
                my_deg += (ull)len;
                if (own && len > DCH) dp[v] = 0;   // chunk items add onto it
            }
        }
        const unsigned nit = (!mover || len == 0) ? 0u : (len > DCH ? (unsigned)((len + DCH - 1) / DCH) : 1u);
        unsigned incl = nit;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned y = __shfl_up_sync(FULLMASK, incl, o);
            if (lane >= o) incl += y;
        }
        if (threadIdx.x == 0) { s_cnt = 0; s_items = 0; }
        __syncthreads();
        const unsigned mm = __ballot_sync(FULLMASK, mover);
        if (mm && lane == 0) atomicAdd(&s_cnt, (unsigned)__popc(mm));
        unsigned ioff = 0;
        const unsigned wtot = __shfl_sync(FULLMASK, incl, 31);
        if (lane == 31 && wtot) ioff = atomicAdd(&s_items, wtot);
        ioff = __shfl_sync(FULLMASK, ioff, 31) + incl - nit;
        __syncthreads();
        if (threadIdx.x == 0) {
            if (s_cnt) atomicAdd(&ctr->n_moved, (ull)s_cnt);
            s_ibase = s_items ? atomicAdd(&ctr->n_items, (ull)s_items) : 0;
        }
        __syncthreads();
        for (unsigned k = 0; k < nit; ++k) {
            const ull at = s_ibase + ioff + k;
            it_v[at] = v;
            it_old[at] = oc;
            it_chunk[at] = (int32_t)k;
        }
        __syncthreads();
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) my_deg += __shfl_xor_sync(FULLMASK, my_deg, o);
    if (lane == 0 && my_deg) atomicAdd(&ctr->moved_deg, my_deg);
}

// §3.5 across ranks, warp per item: owned mover u recomputes d'(u) from its own row and
// pushes -w / +w to its unmoved OWNED neighbours in its old / new community; a remote mover
// pushes along its mirror row (exactly its owned neighbours).
template <bool UNIT>
__global__ void __launch_bounds__(256) k_fab_dp_delta(IterCounters* __restrict__ ctr, const int64_t* __restrict__ rp,
                                                      const int32_t* __restrict__ col, const int64_t* __restrict__ w,
                                                      const int64_t* __restrict__ mrp, const int32_t* __restrict__ mcol,
                                                      const int64_t* __restrict__ mw, const int32_t* __restrict__ C,
                                                      const int32_t* __restrict__ it_v, const int32_t* __restrict__ it_old,
                                                      const int32_t* __restrict__ it_chunk,
                                                      const int32_t* __restrict__ stamp, int64_t* __restrict__ dp,
                                                      const Carry* __restrict__ carry, long long nnz_own, int mode,
                                                      long long lv0, long long lv1, int den) {
    if (!use_delta(ctr, nnz_own, mode, 1, den)) return;
    if (blockIdx.x == 0 && threadIdx.x == 0) ctr->delta_used = 1;
    const int iter_id = carry->iter;
    const int lane = lane_id();
    const long long m = (long long)ctr->n_items;
    const long long wid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long i = wid; i < m; i += nw) {
        const int u = it_v[i], oc = it_old[i], ch = it_chunk[i];
        const int nc = C[u];
        const bool own = u >= lv0 && u < lv1;
        const int64_t* RP = own ? rp : mrp;
        const int32_t* CO = own ? col : mcol;
        const int64_t* WW = own ? w : mw;
        const int64_t rb = RP[u], re = RP[u + 1];
        const bool heavy = re - rb > DCH;
        const int64_t b = rb + (int64_t)ch * DCH, e = heavy ? min(b + DCH, re) : re;
        long long acc = 0;
        for (int64_t j0 = b; j0 < e; j0 += 128) {
            int x[4], cx[4], sx[4];
            long long wt[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int64_t j = j0 + lane + 32 * t;
                x[t] = j < e ? CO[j] : u;
                wt[t] = (UNIT || j >= e) ? 1 : WW[j];
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                cx[t] = x[t] != u ? C[x[t]] : -1;
                sx[t] = x[t] != u ? stamp[x[t]] : iter_id;
            }
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (x[t] == u) continue;
                if (cx[t] == nc) acc += wt[t];
                const bool xown = x[t] >= lv0 && x[t] < lv1;
                if (xown && sx[t] != iter_id) {
                    if (cx[t] == oc) atomicAdd(reinterpret_cast<ull*>(&dp[x[t]]), (ull)(-wt[t]));
                    else if (cx[t] == nc) atomicAdd(reinterpret_cast<ull*>(&dp[x[t]]), (ull)wt[t]);
                }
            }
        }
        if (!own) continue;
        acc = warp_sum_ll(acc);
        if (lane == 0) {
            if (heavy) { if (acc) atomicAdd(reinterpret_cast<ull*>(&dp[u]), (ull)acc); }
            else dp[u] = acc;
        }
    }
}

// this rank's scalars [sum(d'+s) owned, active, pruned, edges scanned, distinct, own moves]
// into every rank's scalar slot
__global__ void k_fab_scal(FabDev f, const Carry* __restrict__ carry, const IterCounters* __restrict__ ctr,
                           const ull* __restrict__ lcount, int level_start) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const int par = level_start ? 0 : fab_par(carry);
    long long v[FAB_NSCAL] = {0};
    v[0] = carry->sumDC;
    if (!level_start) {
        long long sd = 0, sk = 0;
        for (int b = 0; b < NBINS; ++b) { sd += (long long)ctr->bin_deg[b]; sk += (long long)ctr->bin_k[b]; }
        v[1] = (long long)ctr->n_active;
        v[2] = (long long)ctr->n_pruned;
        v[3] = sd;
        v[4] = sk;
        v[5] = (long long)*lcount;
    }
    for (int p = 0; p < f.P; ++p) {
        long long* dst = f.scal[p] + ((long long)par * FAB_MAXP + f.rank) * FAB_NSCAL;
        for (int k = 0; k < FAB_NSCAL; ++k) dst[k] = v[k];
    }
    __threadfence_system();
}

// rank-ordered sums -> N' = qW sum(d'+s) - p S2 (S2 from the replicated Sigma_tot), the
// convergence test (mode 1; Alg. 1 lines 12-13, reading c6/c7), the device log and the loop
// condition; clears the iteration counters and the local move count for the next iteration.
__global__ void k_fab_finish(FabDev f, IterCounters* __restrict__ ctr, Carry* __restrict__ carry,
                             ull* __restrict__ lcount, long long qW_hi, ull qW_lo, long long p, long long T_hi,
                             ull T_lo, int mode, IterLog* __restrict__ log, int log_cap, int max_iters,
                             unsigned long long cond_handle) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const int par = mode == 0 ? 0 : fab_par(carry);
    long long tot[FAB_NSCAL] = {0};
    for (int s = 0; s < f.P; ++s) {
        const long long* src = f.scal[f.rank] + ((long long)par * FAB_MAXP + s) * FAB_NSCAL;
        for (int k = 0; k < FAB_NSCAL; ++k) tot[k] += src[k];
    }
    const i128 S2 = mk128(carry->S2_hi, carry->S2_lo);
    const i128 Nn = mk128(qW_hi, qW_lo) * (i128)tot[0] - (i128)p * S2;
    const i128 N = mk128(carry->N_hi, carry->N_lo);
    int conv = 0;
    if (mode == 1) conv = (ctr->n_moved == 0) || (Nn - N < mk128(T_hi, T_lo)) || *f.err;
    carry->N_prev_hi = hi128(N);
    carry->N_prev_lo = lo128(N);
    carry->N_hi = hi128(Nn);
    carry->N_lo = lo128(Nn);
    carry->sumDC = tot[0];
    carry->converged = conv;
    carry->t_ns = globaltimer_ns();
    if (mode == 0) return;
    ctr->n_active = (ull)tot[1];
    ctr->n_pruned = (ull)tot[2];
    for (int b = 0; b < NBINS; ++b) { ctr->bin_deg[b] = 0; ctr->bin_k[b] = 0; }
    ctr->bin_deg[0] = (ull)tot[3];
    ctr->bin_k[0] = (ull)tot[4];
    record_iteration(ctr, carry, log, log_cap, max_iters, cond_handle);
    ull* c = reinterpret_cast<ull*>(ctr);
    for (int i = 0; i < (int)(sizeof(IterCounters) / sizeof(ull)); ++i) c[i] = 0;
    *lcount = 0;
}

// mirror block of the owned rows (§8(e)): entry (v, u, w) of an owned row v becomes entry
// (u -> v, w) of mirror row u; counting sort by u
__global__ void k_mirror_count(long long nnz, const int32_t* __restrict__ col, long long* __restrict__ cnt) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (long long)gridDim.x * blockDim.x)
        atomicAdd(reinterpret_cast<ull*>(&cnt[col[i]]), 1ull);
}
__global__ void k_mirror_scatter(long long nnz, const int32_t* __restrict__ row, const int32_t* __restrict__ col,
                                 const int64_t* __restrict__ w, const long long* __restrict__ mrp,
                                 long long* __restrict__ cur, int32_t* __restrict__ mcol, int64_t* __restrict__ mw) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += (long long)gridDim.x * blockDim.x) {
        const int u = col[i];
        const long long o = mrp[u] + (long long)atomicAdd(reinterpret_cast<ull*>(&cur[u]), 1ull);
        mcol[o] = row[i];
        if (w) mw[o] = w[i];
    }
}
