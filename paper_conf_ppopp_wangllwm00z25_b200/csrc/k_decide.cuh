// k_decide.cuh — DecideAndMove kernels (Alg. 1 lines 14-16), §8(a) a3/a4.
//
// Every kernel computes, for each queued (active) vertex v, the exact integer
// decision of reading c1/c4/c5:
//   score(c) = qW d_c(v) - p Sig[c] d(v)          for neighbouring c != C[v]
//   stay     = qW d'(v) - p (Sig[C[v]] - d(v)) d(v)
//   move to argmax (score, lowest c) iff score > stay, unless singleton swap.
// and writes nextC[v] (C[v] to stay).  The kernels differ only in how the
// per-community weights d_c(v) are aggregated:
//   k_decide_sub   (a3) deg <= G lanes: __match_any_sync over the group (Alg. 2)
//   k_decide_warp  (a4) deg <= 32*E: per-warp shared-memory hash table
//   k_decide_block (a4) larger: per-block shared-memory table H0 spilling to a
//                  per-block global table H1 (hierarchical hash, §4.2)
// Hash kernels follow Alg. 3's ownership rule (footnote 2): the thread
// that inserts a community into the table owns it and evaluates its gain once
// all inserts are done, so only occupied slots are ever visited.
//
// Modes (chosen per level by the host, never changing a result):
//   DM_FAST : int64 gains, 32-bit aggregates (W < 2^31), (score, -c) packed in
//             one int64 key so the argmax is a single 64-bit max reduction
//             (needs max(p,q) W maxdeg < 2^(62 - idbits))
//   DM_W64  : int64 gains, 64-bit aggregates, (score, c) pairs
//   DM_W128 : __int128 gains (reading c16), 64-bit aggregates
#pragma once
#include "common.cuh"

enum { DM_FAST = 0, DM_W64 = 1, DM_W128 = 2 };
template <int M> struct ModeT;
template <> struct ModeT<DM_FAST> { typedef long long ST; typedef unsigned VT; static constexpr bool PK = true; };
template <> struct ModeT<DM_W64> { typedef long long ST; typedef unsigned VT; static constexpr bool PK = false; };
template <> struct ModeT<DM_W128> { typedef i128 ST; typedef ull VT; static constexpr bool PK = false; };

// running argmax over (score, -community)
template <typename ST, bool PK> struct Arg {
    ST s;
    int c;
    __device__ __forceinline__ void init(int, long long) { s = st_min<ST>(); c = INT_MAX; }
    __device__ __forceinline__ void offer(ST sc, int cc) { if (better(sc, cc, s, c)) { s = sc; c = cc; } }
    __device__ __forceinline__ void xor_merge(int off) {
        ST os = shfl_xor_st(s, off);
        int oc = __shfl_xor_sync(FULLMASK, c, off);
        if (better(os, oc, s, c)) { s = os; c = oc; }
    }
    __device__ __forceinline__ bool valid() const { return c != INT_MAX; }
    __device__ __forceinline__ ST score() const { return s; }
    __device__ __forceinline__ int comm() const { return c; }
};
template <> struct Arg<long long, true> {
    long long k;
    int bits;
    long long mask;
    __device__ __forceinline__ void init(int idbits, long long idmask) { k = LLONG_MIN; bits = idbits; mask = idmask; }
    __device__ __forceinline__ void offer(long long sc, int cc) {
        long long kk = (long long)((ull)sc << bits) | (mask - cc);
        k = kk > k ? kk : k;
    }
    __device__ __forceinline__ void xor_merge(int off) {
        long long o = __shfl_xor_sync(FULLMASK, k, off);
        k = o > k ? o : k;
    }
    __device__ __forceinline__ bool valid() const { return k != LLONG_MIN; }
    __device__ __forceinline__ long long score() const { return k >> bits; }
    __device__ __forceinline__ int comm() const { return (int)(mask - (k & mask)); }
};

template <typename ST>
__device__ __forceinline__ ST gain(ST qW, ST p, long long wc, long long sig, long long dv) {
    return qW * (ST)wc - p * (ST)sig * (ST)dv;
}

template <typename ST, typename A>
__device__ __forceinline__ int decide_final(int cv, int szv, long long dv, long long own, long long sig_cv,
                                            const A& best, const int32_t* __restrict__ size, ST qW, ST p) {
    ST stay = qW * (ST)own - p * (ST)(sig_cv - dv) * (ST)dv;
    int tgt = cv;
    if (best.valid() && best.score() > stay) {          // strictly better than staying (c4)
        tgt = best.comm();
        if (szv == 1 && tgt > cv && size[tgt] == 1) tgt = cv;   // swap suppression (c5)
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
    int32_t* nextC;     // decision of every processed vertex (C[v] to stay)
    const int32_t* ckey;   // level 0: C[col[e]] per CSR entry (-1 = self loop), rewritten by every full
                           // d' pass; used while *ckey_valid, else C[col[e]] is gathered here
    const int* ckey_valid;
    IterCounters* ctr;
    int check;
    int table_mode;     // block bin's table (§4.2): 0 hierarchical, 1 global-only, 2 unified
    int idbits;         // packed-key layout (DM_FAST)
    long long idmask;
    long long nlev;     // vertices of the level (bound on distinct communities per row)
};

// ---------------------------------------------------------------------------
// a3: sub-warp groups of G lanes, one neighbour per lane (Alg. 2).
// Equal communities are found with __match_any_sync; d_c(v) is popc(peers) on
// unit-weight levels, else the peers' weights summed onto the group leader
// with shared-memory atomics.  Each group handles U independent vertices per
// iteration with all their loads issued before use.
// ---------------------------------------------------------------------------
template <int G, int U, int M, bool UNIT>
__device__ __forceinline__ unsigned decide_sub_bin(QView queue, int bin, const DecideArgs& a,
                                                   typename ModeT<M>::ST qW, typename ModeT<M>::ST p,
                                                   typename ModeT<M>::VT (*s_acc)[32]) {
    typedef typename ModeT<M>::ST ST;
    typedef typename ModeT<M>::VT VT;
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const int gid = lane / G, gl = lane % G;
    const unsigned gmask = (G == 32) ? FULLMASK : (((1u << G) - 1u) << (gid * G));
    const int glead = gid * G;
    const long long count = (long long)a.ctr->bin_count[bin];
    const long long nwarps = (long long)gridDim.x * (blockDim.x >> 5);
    const long long per = (32 / G) * U;
    unsigned my_k = 0;
    for (long long base = ((long long)blockIdx.x * (blockDim.x >> 5) + wib) * per; base < count;
         base += nwarps * per) {
        QRec q[U];
        int u[U], cu[U];
        long long wt[U];
        bool valid[U], has[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            long long i = base + (long long)k * (32 / G) + gid;
            valid[k] = i < count;
            if (valid[k]) q[k] = queue[i];
            else { q[k].v = 0; q[k].deg = 0; q[k].beg = 0; q[k].cv = -2; q[k].szv = 0; q[k].dv = 0; q[k].sigv = 0; }
        }
        if (a.ckey) {   // neighbour communities read straight from the per-entry array
#pragma unroll
            for (int k = 0; k < U; ++k) {
                has[k] = valid[k] && gl < q[k].deg;
                u[k] = has[k] ? a.ckey[q[k].beg + gl] : -1;
                wt[k] = (has[k] && !UNIT) ? a.w[q[k].beg + gl] : 1;
            }
#pragma unroll
            for (int k = 0; k < U; ++k) {
                if (u[k] < 0) has[k] = false;                 // self loop is not a neighbour
                cu[k] = has[k] ? u[k] : (-1 - lane);
            }
        } else {
#pragma unroll
            for (int k = 0; k < U; ++k) {
                has[k] = valid[k] && gl < q[k].deg;
                u[k] = has[k] ? a.col[q[k].beg + gl] : -1;
                wt[k] = (has[k] && !UNIT) ? a.w[q[k].beg + gl] : 1;
            }
#pragma unroll
            for (int k = 0; k < U; ++k) {
                if (u[k] == q[k].v) has[k] = false;           // self loop is not a neighbour
                cu[k] = has[k] ? a.C[u[k]] : (-1 - lane);     // unique sentinel per empty lane
            }
        }
        unsigned peers[U];
        bool isL[U];
        long long sig[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            peers[k] = __match_any_sync(FULLMASK, cu[k]) & gmask;
            isL[k] = has[k] && lane == __ffs(peers[k]) - 1;
            sig[k] = (isL[k] && cu[k] != q[k].cv) ? a.Sig[cu[k]] : 0;
        }
        int tgt[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            long long wc, own;
            if (UNIT) {
                wc = __popc(peers[k]);
                own = __popc(__ballot_sync(FULLMASK, has[k] && cu[k] == q[k].cv) & gmask);
            } else {
                wc = (long long)group_sum(peers[k], has[k] ? (VT)wt[k] : (VT)0, s_acc[wib]);
                unsigned om = __ballot_sync(FULLMASK, isL[k] && cu[k] == q[k].cv) & gmask;
                long long wl = __shfl_sync(FULLMASK, wc, om ? __ffs(om) - 1 : 0);
                own = om ? wl : 0;
            }
            my_k += isL[k];
            Arg<ST, ModeT<M>::PK> best;
            best.init(a.idbits, a.idmask);
            if (isL[k] && cu[k] != q[k].cv) best.offer(gain<ST>(qW, p, wc, sig[k], q[k].dv), cu[k]);
#pragma unroll
            for (int off = G / 2; off > 0; off >>= 1) best.xor_merge(off);
            tgt[k] = q[k].cv;
            if (valid[k] && lane == glead) {
                if (a.check && own != a.dp[q[k].v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
                tgt[k] = decide_final<ST>(q[k].cv, q[k].szv, q[k].dv, own, q[k].sigv, best, a.size, qW, p);
            }
        }
#pragma unroll
        for (int k = 0; k < U; ++k)
            if (valid[k] && gl == 0) a.nextC[q[k].v] = tgt[k];
    }
    return my_k;
}

// bins 0-3 (rows <= 4, 8, 16, 32) in one launch: the block's warps sweep each
// bin with its own group size, so empty bins cost nothing
#ifndef GALA_EARLY_EXIT
#define GALA_EARLY_EXIT 1   // blocks without work return before their table clears (late, mostly pruned iterations)
#endif
#ifndef GALA_SMALL_MINB
#define GALA_SMALL_MINB 4   // <= 64 registers: 32 warps per SM (measured -30% vs 72-80 regs)
#endif
#ifndef GALA_WARP_SCAN
#define GALA_WARP_SCAN 0   // warp128: evaluate by scanning the 256-slot table instead of keeping a distinct list
#endif
#ifndef GALA_WARP_KV
#define GALA_WARP_KV 1   // warp kernels: packed 64-bit (key, sum) table slots, batched list evaluation
#endif
#ifndef GALA_WARP_PREFETCH
#define GALA_WARP_PREFETCH 1   // warp128: next vertex's row loaded during this one's evaluation
#endif
#ifndef GALA_WARP_MINB
#define GALA_WARP_MINB 4   // <= 64 registers (an explicit min of 1 lets ptxas take 80)
#endif
#ifndef GALA_W512_MINB
#define GALA_W512_MINB 4   // 128 regs, 4 blocks of 128 threads
#endif
#ifndef GALA_SINGLE_MINB
#define GALA_SINGLE_MINB 1
#endif
#ifndef GALA_U16
#define GALA_U16 4
#endif
#ifndef GALA_U32
#define GALA_U32 4
#endif
template <int M, bool UNIT>
__global__ void __launch_bounds__(256, GALA_SMALL_MINB) k_decide_small(QRec* queues, long long qstride,
                                                      DecideArgs a, typename ModeT<M>::ST qW,
                                                      typename ModeT<M>::ST p) {
    __shared__ typename ModeT<M>::VT s_acc[8][32];
#if GALA_EARLY_EXIT
    {   // first record of this block in each sub-bin (G lanes per vertex, U vertices per group, 8 warps)
        const long long b0 = (long long)blockIdx.x * 8;
        if (b0 * 8 * 4 >= (long long)a.ctr->bin_count[BIN_S4] && b0 * 4 * 4 >= (long long)a.ctr->bin_count[BIN_S8] &&
            b0 * 2 * GALA_U16 >= (long long)a.ctr->bin_count[BIN_S16] &&
            b0 * GALA_U32 >= (long long)a.ctr->bin_count[BIN_S32])
            return;
    }
#endif
    if (a.ckey && !*a.ckey_valid) a.ckey = nullptr;
    unsigned k0 = decide_sub_bin<4, 4, M, UNIT>(qview(queues, qstride, BIN_S4), BIN_S4, a, qW, p, s_acc);
    unsigned k1 = decide_sub_bin<8, 4, M, UNIT>(qview(queues, qstride, BIN_S8), BIN_S8, a, qW, p, s_acc);
    unsigned k2 = decide_sub_bin<16, GALA_U16, M, UNIT>(qview(queues, qstride, BIN_S16), BIN_S16, a, qW, p, s_acc);
    unsigned k3 = decide_sub_bin<32, GALA_U32, M, UNIT>(qview(queues, qstride, BIN_S32), BIN_S32, a, qW, p, s_acc);
    const unsigned kk[4] = {k0, k1, k2, k3};
#pragma unroll
    for (int b = 0; b < 4; ++b) {
        ull t = block_sum_ull<256>((ull)kk[b]);
        if (threadIdx.x == 0 && t) atomicAdd(&a.ctr->bin_k[b], t);
    }
}

// ---------------------------------------------------------------------------
// open-addressing insert of (c, +w): CAS on the key, atomicAdd on the value
// (Alg. 3 lines 6-10).  Linear probing over at most `win` slots.
// Returns the slot and sets *fresh when this thread created the key; returns
// -1 when the window holds only other keys.
// ---------------------------------------------------------------------------
template <typename VT>
__device__ __forceinline__ int ht_insert(int c, VT wt, int* keys, VT* vals, unsigned mask, unsigned h, int win,
                                         bool* fresh) {
    *fresh = false;
    for (int t = 0; t < win; ++t) {
        int k = *(volatile int*)&keys[h];
        if (k == -1) {
            int old = atomicCAS(&keys[h], -1, c);
            if (old == -1) { *fresh = true; atomicAdd(&vals[h], wt); return (int)h; }
            if (old == c) { atomicAdd(&vals[h], wt); return (int)h; }
        } else if (k == c) {
            atomicAdd(&vals[h], wt);
            return (int)h;
        }
        h = (h + 1) & mask;
    }
    return -1;
}

// Bucketed form of the same linear probe: slots are read four at a time (one
// 16-byte load of an aligned 4-key bucket, starting at the bucket holding h)
// and the empty slots of a bucket are claimed in slot order, so the probe
// sequence -- and therefore every result -- is that of slot-wise linear
// probing from the bucket start.  Cuts the divergent probe loop of the lane
// with the longest chain (which the whole warp waits for) about 4x.  Needs a
// 16-byte-aligned key array and mask >= 3; `win` is rounded up to buckets.
template <typename VT, bool SH>
__device__ __forceinline__ int ht_insert4(int c, VT wt, int* keys, VT* vals, unsigned mask, unsigned h, int win,
                                          bool* fresh) {
    if (mask < 3) return ht_insert<VT>(c, wt, keys, vals, mask, h, win, fresh);
    *fresh = false;
    unsigned b = h & ~3u;
    const int nb = (win + 3) >> 2;
    for (int t = 0; t < nb; ++t) {
        const int4 k4 = ld_bucket<SH>(keys + b);
        const unsigned hit = match4(k4, c);
        if (hit) {
            const unsigned s = b + __ffs(hit) - 1;
            atomicAdd(&vals[s], wt);
            return (int)s;
        }
        for (unsigned em = match4(k4, -1); em; em &= em - 1) {   // empties in slot order
            const unsigned s = b + __ffs(em) - 1;
            const int old = atomicCAS(&keys[s], -1, c);
            if (old == -1 || old == c) {
                *fresh = old == -1;
                atomicAdd(&vals[s], wt);
                return (int)s;
            }
        }
        b = (b + 4) & mask;
    }
    return -1;
}

// Packed form for 32-bit aggregates: one 64-bit word per slot, key in the high half, the
// weight sum in the low half (KV_EMPTY = key -1, sum 0).  A fresh key is created with ONE
// 64-bit CAS that also stores its first sum; an existing key takes a native 32-bit add on the
// low half (the sum never reaches 2^32: it is at most W < 2^31 on these levels).  Same
// slot-wise linear probe, hence the same table contents as ht_insert.
#define KV_EMPTY 0xFFFFFFFF00000000ull
__device__ __forceinline__ int kv_insert(int c, unsigned wt, ull* tbl, unsigned mask, unsigned h, int win, bool* fresh) {
    *fresh = false;
    const ull mine = ((ull)(unsigned)c << 32) | wt;
    for (int t = 0; t < win; ++t) {
        ull k = *(volatile ull*)&tbl[h];
        if (k == KV_EMPTY) {
            k = atomicCAS(&tbl[h], KV_EMPTY, mine);
            if (k == KV_EMPTY) { *fresh = true; return (int)h; }
        }
        if ((int)(k >> 32) == c) {
            atomicAdd(reinterpret_cast<unsigned*>(&tbl[h]), wt);   // low half (little endian)
            return (int)h;
        }
        h = (h + 1) & mask;
    }
    return -1;
}

// ---------------------------------------------------------------------------
// a4 (mid degree): one warp per vertex (deg <= MAXDEG), per-warp shared-memory
// table of 2*MAXDEG slots (load <= 1/2, never spills) and a distinct-key list.
// Rows are loaded 4 entries per lane at a time (4 independent gathers in
// flight per lane).  The table is cleared once per kernel; every vertex clears
// exactly the slots it used.  Dynamic shared memory: WPB warps per block.
// ---------------------------------------------------------------------------
template <int GW, int MAXDEG, int M>
struct WarpSmem {
    static constexpr int WCAP = 2 * MAXDEG;                 // table slots per group (load <= 1/2)
    static constexpr int WPB = MAXDEG <= 128 ? 8 : 4;       // warps per block
    static constexpr size_t per_group =
        (size_t)WCAP * (sizeof(int) + sizeof(typename ModeT<M>::VT)) + (size_t)MAXDEG * sizeof(short) + 16;
    static constexpr size_t per_warp = 32 * sizeof(ull) + per_group * (32 / GW);
    static constexpr size_t bytes = per_warp * WPB;
};

// GW lanes (16 or 32) per vertex, deg <= MAXDEG = 4 * GW; 32/GW vertices per warp
template <int GW, int MAXDEG, int M, bool UNIT>
__global__ void __launch_bounds__(32 * WarpSmem<GW, MAXDEG, M>::WPB, MAXDEG <= 128 ? GALA_WARP_MINB : GALA_W512_MINB) k_decide_warp(QView queue,
                                                                                  int bin, DecideArgs a,
                                                                                  typename ModeT<M>::ST qW,
                                                                                  typename ModeT<M>::ST p) {
    if (a.ckey && !*a.ckey_valid) a.ckey = nullptr;
    typedef typename ModeT<M>::ST ST;
    typedef typename ModeT<M>::VT VT;
    typedef WarpSmem<GW, MAXDEG, M> SM;
    constexpr int WCAP = SM::WCAP;
    constexpr unsigned WMASK = WCAP - 1;
    constexpr int CH = MAXDEG / GW;   // entries per lane per round
    constexpr int NG = 32 / GW;       // vertices per warp
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const long long count = (long long)a.ctr->bin_count[bin];
#if GALA_EARLY_EXIT
    if ((long long)blockIdx.x * SM::WPB * NG >= count) return;   // no vertex for this block: skip the table clear
#endif
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const int gid = lane / GW, gl = lane % GW;
    const unsigned gmask = GW == 32 ? FULLMASK : (((1u << GW) - 1u) << (gid * GW));
    unsigned char* wbase = smem_raw + SM::per_warp * wib;
    VT* scratch = reinterpret_cast<VT*>(wbase);
    unsigned char* base = wbase + 32 * sizeof(ull) + SM::per_group * gid;
    VT* vals = reinterpret_cast<VT*>(base);
    int* keys = reinterpret_cast<int*>(base + (size_t)WCAP * sizeof(VT));
    short* list = reinterpret_cast<short*>(base + (size_t)WCAP * (sizeof(VT) + sizeof(int)));
    int* cnt = reinterpret_cast<int*>(base + (size_t)WCAP * (sizeof(VT) + sizeof(int)) + (size_t)MAXDEG * sizeof(short));
    // KV: packed 64-bit (key, 32-bit sum) slots over the same bytes as keys + vals
    constexpr bool KV = GALA_WARP_KV && sizeof(VT) == 4 && !(GALA_WARP_SCAN && MAXDEG <= 128);
    ull* tbl = reinterpret_cast<ull*>(base);
    if (KV) { for (int j = gl; j < WCAP; j += GW) tbl[j] = KV_EMPTY; }
    else { for (int j = gl; j < WCAP; j += GW) { keys[j] = -1; vals[j] = 0; } }
    if (gl == 0) *cnt = 0;
    __syncwarp();
    const long long nwarps = (long long)gridDim.x * SM::WPB;
    unsigned my_k = 0;
    long long base_i = ((long long)blockIdx.x * SM::WPB + wib) * NG;
    // PF: the row entries of a group's NEXT vertex are loaded while the current one is
    // evaluated (every row here fits one round: deg <= MAXDEG = GW * CH)
    constexpr bool PF = GALA_WARP_PREFETCH && MAXDEG <= 128 && MAXDEG == GW * CH;
    constexpr bool SCAN = GALA_WARP_SCAN && MAXDEG <= 128;   // table scan instead of a distinct list
    const int* __restrict__ rsrc = a.ckey ? a.ckey : a.col;
    int pu[CH];
    VT pw[CH];
    QRec qn;
    if (base_i + gid < count) qn = queue[base_i + gid];
    if (PF) {
        const bool ok = base_i + gid < count;
#pragma unroll
        for (int k = 0; k < CH; ++k) {
            const int j = gl + GW * k;
            pu[k] = ok && j < qn.deg ? rsrc[qn.beg + j] : -1;
            pw[k] = (ok && j < qn.deg && !UNIT) ? (VT)a.w[qn.beg + j] : (VT)1;
        }
    }
    for (; base_i < count; base_i += nwarps * NG) {            // warp-uniform
        const bool valid = base_i + gid < count;
        const QRec q = qn;
        const int v = valid ? q.v : 0, deg = valid ? q.deg : 0, cv = valid ? q.cv : -2;
        const int64_t beg = valid ? q.beg : 0;
        const long long dv = valid ? q.dv : 0, sig_cv = valid ? q.sigv : 0;
        const long long inext = base_i + nwarps * NG + gid;
        if (inext < count) qn = queue[inext];                  // prefetch the next record
        int dmax = deg;
#pragma unroll
        for (int o = 16; o >= GW; o >>= 1) dmax = max(dmax, __shfl_xor_sync(FULLMASK, dmax, o));
        long long own = 0;   // the own community only feeds d'(v): summed in registers, never inserted
        for (int r0 = 0; r0 < dmax; r0 += GW * CH) {           // warp-uniform rounds
            int uu[CH];
            VT ww[CH];
            int cc[CH];
            if (PF) {
#pragma unroll
                for (int k = 0; k < CH; ++k) { uu[k] = pu[k]; ww[k] = pw[k]; }
            } else {
#pragma unroll
                for (int k = 0; k < CH; ++k) {
                    int j = r0 + gl + GW * k;
                    uu[k] = j < deg ? rsrc[beg + j] : -1;
                    ww[k] = (j < deg && !UNIT) ? (VT)a.w[beg + j] : (VT)1;
                }
            }
            if (a.ckey) {
#pragma unroll
                for (int k = 0; k < CH; ++k) cc[k] = uu[k];
            } else {
#pragma unroll
                for (int k = 0; k < CH; ++k) cc[k] = (uu[k] >= 0 && uu[k] != v) ? a.C[uu[k]] : -1;
            }
#pragma unroll
            for (int k = 0; k < CH; ++k)
                if (cc[k] == cv) { own += (long long)ww[k]; cc[k] = -1; }
#pragma unroll
            for (int k = 0; k < CH; ++k) {
                if (r0 + GW * k >= dmax) break;                // warp-uniform
                // combine equal communities of this chunk first (one insert per community)
                const unsigned peers = __match_any_sync(FULLMASK, cc[k] >= 0 ? cc[k] : -1 - lane) & gmask;
                const VT sum = UNIT ? (VT)__popc(peers) : group_sum(peers, cc[k] >= 0 ? ww[k] : (VT)0, scratch);
                bool fresh = false;
                int slot = -1;
                if (cc[k] >= 0 && lane == __ffs(peers) - 1) {
                    if (KV) slot = kv_insert(cc[k], (unsigned)sum, tbl, WMASK, hash_slot(cc[k], WMASK), WCAP, &fresh);
                    else slot = MAXDEG > 128   // bucketed probing pays only in the larger tables (measured)
                               ? ht_insert4<VT, true>(cc[k], sum, keys, vals, WMASK, hash_slot(cc[k], WMASK), WCAP, &fresh)
                               : ht_insert<VT>(cc[k], sum, keys, vals, WMASK, hash_slot(cc[k], WMASK), WCAP, &fresh);
                }
                if (!SCAN) append_fresh<short>(fresh, slot, gmask, cnt, list);
            }
        }
        if (PF) {   // next vertex's row: in flight during this vertex's evaluation
            const bool ok = inext < count;
#pragma unroll
            for (int k = 0; k < CH; ++k) {
                const int j = gl + GW * k;
                pu[k] = ok && j < qn.deg ? rsrc[qn.beg + j] : -1;
                pw[k] = (ok && j < qn.deg && !UNIT) ? (VT)a.w[qn.beg + j] : (VT)1;
            }
        }
        __syncwarp();
        Arg<ST, ModeT<M>::PK> best;
        best.init(a.idbits, a.idmask);
        if (SCAN) {   // no distinct list: the group scans its whole table (4 slots per 16-byte load)
            for (int t0 = gl * 4; t0 < WCAP; t0 += GW * 4) {
                const int4 k4 = *reinterpret_cast<const int4*>(keys + t0);
                if ((k4.x & k4.y & k4.z & k4.w) == -1) continue;   // all four empty
                const int cs[4] = {k4.x, k4.y, k4.z, k4.w};
                long long ws[4], sg[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    ws[k] = cs[k] >= 0 ? (long long)vals[t0 + k] : 0;
                    sg[k] = (cs[k] >= 0 && cs[k] != cv) ? a.Sig[cs[k]] : 0;
                }
                *reinterpret_cast<int4*>(keys + t0) = make_int4(-1, -1, -1, -1);
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    if (cs[k] < 0) continue;
                    vals[t0 + k] = 0;
                    ++my_k;
                    if (cs[k] == cv) own = ws[k];
                    else best.offer(gain<ST>(qW, p, ws[k], sg[k], dv), cs[k]);
                }
            }
        }
        const int m = SCAN ? 0 : *cnt;
        my_k += (!SCAN && gl == 0) ? m : 0;
        // KV: the group's distinct list in batches of 4 slots per lane, the batch count bounded
        // by the group's own list length (no predicated-off batches)
        for (int b0 = 0; KV && b0 < m; b0 += GW * 4) {
            int cs[4];
            unsigned ws[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                cs[k] = -1;
                ws[k] = 0;
                const int t = b0 + gl + GW * k;
                if (b0 + GW * k < m && t < m) {
                    const int slot = list[t];
                    const ull kv = tbl[slot];
                    tbl[slot] = KV_EMPTY;
                    cs[k] = (int)(kv >> 32);
                    ws[k] = (unsigned)kv;
                }
            }
            long long sg[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) sg[k] = cs[k] >= 0 ? a.Sig[cs[k]] : 0;
#pragma unroll
            for (int k = 0; k < 4; ++k)
                if (cs[k] >= 0) best.offer(gain<ST>(qW, p, (long long)ws[k], sg[k], dv), cs[k]);
        }
        for (int t0 = gl; !KV && t0 < m; t0 += GW * CH) {
            int cs[CH];
            long long ws[CH];
#pragma unroll
            for (int k = 0; k < CH; ++k) {
                int t = t0 + GW * k;
                cs[k] = -1;
                ws[k] = 0;
                if (t < m) {
                    int slot = list[t];
                    cs[k] = keys[slot];
                    ws[k] = (long long)vals[slot];
                    keys[slot] = -1;
                    vals[slot] = 0;
                }
            }
            long long sg[CH];
#pragma unroll
            for (int k = 0; k < CH; ++k) sg[k] = (cs[k] >= 0 && cs[k] != cv) ? a.Sig[cs[k]] : 0;
#pragma unroll
            for (int k = 0; k < CH; ++k) {
                if (cs[k] < 0) continue;
                if (cs[k] == cv) own = ws[k];
                else best.offer(gain<ST>(qW, p, ws[k], sg[k], dv), cs[k]);
            }
        }
        __syncwarp();
        if (gl == 0) *cnt = 0;
#pragma unroll
        for (int off = GW / 2; off > 0; off >>= 1) {
            best.xor_merge(off);
            own += __shfl_xor_sync(FULLMASK, own, off);
        }
        if (valid && gl == 0) {
            if (a.check && own != a.dp[v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            a.nextC[v] = decide_final<ST>(cv, q.szv, dv, own, sig_cv, best, a.size, qW, p);
            my_k += own ? 1u : 0u;
        }
        __syncwarp();
    }
    ull k = block_sum_ull<32 * SM::WPB>((ull)my_k);
    if (threadIdx.x == 0 && k) atomicAdd(&a.ctr->bin_k[bin], k);
}

// ---------------------------------------------------------------------------
// a4 (high degree / hubs): one block per vertex, hierarchical table (§4.2
// "Hierarchical"): shared-memory H0 (smem_cap slots, probed over a
// window of HWIN slots when the row cannot fit at load 1/2), overflow to the
// block's global H1 with linear probing.  New keys are appended to a distinct
// list (shared memory for H0, global for H1); after the inserts each list
// entry is evaluated and its slot cleared, so both tables stay empty between
// vertices.  Vertices are fetched dynamically; each thread batches E entries.
// ---------------------------------------------------------------------------
#define HWIN 16
// CLS 0: every queued vertex; CLS 1: rows <= split only; CLS 2: rows > split only (two launches
// with arenas sized for their class: short rows get small blocks, more vertices in flight per SM).
// A class kernel fetches the queue in batches of FETCH_B indices (thread 0) and skips the rows of
// the other class.
#define FETCH_B 8
template <int CLS>
__device__ __forceinline__ long long block_next_item(QView queue, long long count, ull* cursor, int split,
                                                     int* s_batch, int* s_nb, int* s_bi) {
    if (CLS == 0) return (long long)atomicAdd(cursor, 1ull);
    for (;;) {
        if (*s_bi < *s_nb) return s_batch[(*s_bi)++];
        const long long b0 = (long long)atomicAdd(cursor, (ull)FETCH_B);
        if (b0 >= count) return count;
        int dg[FETCH_B];
#pragma unroll
        for (int t = 0; t < FETCH_B; ++t) dg[t] = b0 + t < count ? queue[b0 + t].deg : -1;
        int nb = 0;
#pragma unroll
        for (int t = 0; t < FETCH_B; ++t)
            if (dg[t] >= 0 && ((dg[t] <= split) == (CLS == 1))) s_batch[nb++] = (int)(b0 + t);
        *s_nb = nb;
        *s_bi = 0;
    }
}

#ifndef GALA_BLOCK_MINB
#define GALA_BLOCK_MINB 0      // >0: min resident 512-thread blocks per SM of the long-row class (register cap);
                               // 0: no bound (an explicit 1 lets ptxas take 75-100 registers and halves occupancy)
#endif
#ifndef GALA_BLOCK_NEXT
#define GALA_BLOCK_NEXT 1      // the next vertex is fetched while the current one is processed
#endif
#ifndef GALA_BLOCK_PIPE
#define GALA_BLOCK_PIPE 1      // the next round's row entries are loaded while the current round is inserted
#endif
#if GALA_BLOCK_MINB > 0
#define BLOCK_LB(BT) __launch_bounds__(BT, BT >= 512 ? GALA_BLOCK_MINB : 1)
#else
#define BLOCK_LB(BT) __launch_bounds__(BT)
#endif
template <int BT, int E, int M, bool UNIT, int CLS = 0>
__global__ void BLOCK_LB(BT) k_decide_block(QView queue, int bin, DecideArgs a,
                                                     typename ModeT<M>::ST qW, typename ModeT<M>::ST p, int smem_cap,
                                                     int* __restrict__ gkeys_all, ull* __restrict__ gvals_all,
                                                     int* __restrict__ glist_all, long long gcap, int split = 0) {
    if (a.ckey && !*a.ckey_valid) a.ckey = nullptr;
    typedef typename ModeT<M>::ST ST;
    typedef typename ModeT<M>::VT VT;
    typedef Arg<ST, ModeT<M>::PK> A;
    // H0 = keys + values only (no distinct list: the table prefix a vertex used is
    // scanned instead, <= 4 slots per row entry), so more blocks fit per SM
    extern __shared__ __align__(16) unsigned char smem_raw[];
    VT* vals = reinterpret_cast<VT*>(smem_raw);
    int* keys = reinterpret_cast<int*>(smem_raw + (size_t)smem_cap * sizeof(VT));
    __shared__ long long s_item;
    __shared__ int s_gcnt;
    __shared__ A r_a[BT / 32];
    __shared__ long long r_own[BT / 32];
    __shared__ VT s_scr[BT / 32][32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    int* gkeys = gkeys_all + (long long)blockIdx.x * gcap;
    ull* gvals = gvals_all + (long long)blockIdx.x * gcap;
    int* glist = glist_all + (long long)blockIdx.x * gcap;
    const long long count = (long long)a.ctr->bin_count[bin];
#if GALA_EARLY_EXIT
    // items are claimed from a shared cursor, so blocks 0..count-1 can take them all:
    // the rest leave before clearing their arena
    if ((long long)blockIdx.x >= count) return;
#endif
    for (int j = threadIdx.x; j < smem_cap; j += BT) { keys[j] = -1; vals[j] = 0; }
    if (threadIdx.x == 0) s_gcnt = 0;
    unsigned my_k = 0;
    ull my_h0 = 0, my_h1 = 0, my_k0 = 0, my_k1 = 0;   // table access / maintenance counters (§4.2)
    __shared__ int s_batch[FETCH_B], s_nb, s_bi;
    if (threadIdx.x == 0) { s_nb = 0; s_bi = 0; }
    ull* const cursor = CLS == 2 ? &a.ctr->cursor_hi : &a.ctr->cursor[bin];
    // NEXT: the next item is fetched by thread 0 while the block works on the current one (its
    // cursor atomic and queue loads are off the per-vertex critical path)
    // (with its queue record: the block reads the current record from shared memory)
    __shared__ long long s_next;
    __shared__ QRec s_q, s_qn;
    if (GALA_BLOCK_NEXT && threadIdx.x == 0) {
        s_next = block_next_item<CLS>(queue, count, cursor, split, s_batch, &s_nb, &s_bi);
        if (s_next < count) s_qn = queue[s_next];
    }
    for (;;) {
        if (threadIdx.x == 0) {
            if (GALA_BLOCK_NEXT) { s_item = s_next; s_q = s_qn; }
            else s_item = block_next_item<CLS>(queue, count, cursor, split, s_batch, &s_nb, &s_bi);
        }
        __syncthreads();
        long long i = s_item;
        if (i >= count) break;
        const QRec q = GALA_BLOCK_NEXT ? s_q : queue[i];
        if (GALA_BLOCK_NEXT && threadIdx.x == 0) {
            s_next = block_next_item<CLS>(queue, count, cursor, split, s_batch, &s_nb, &s_bi);
            if (s_next < count) s_qn = queue[s_next];
        }
        const int v = q.v, deg = q.deg, cv = q.cv;
        const int64_t beg = q.beg;
        long long own = 0;   // the own community only feeds d'(v): summed in registers, never inserted
        // H0 prefix used by this vertex: nextpow2(2 deg) slots (load <= 1/2, never spills)
        // when that fits, else the whole arena probed over a window of HWIN slots
        const int need = deg > 32 ? (int)(1u << (32 - __clz(2 * deg - 1))) : 64;
        const int tcap = need <= smem_cap ? need : smem_cap;
        const int win = need <= smem_cap ? tcap : HWIN;
        const unsigned smask = (unsigned)tcap - 1;
        long long gc = deg > 32 ? (1LL << (64 - __clzll(2LL * deg - 1))) : 64;   // H1 slots
        if (gc > gcap) gc = gcap;
        const unsigned gmask = (unsigned)gc - 1;
        int uu[E];
        VT ww[E];
#pragma unroll
        for (int k = 0; k < E; ++k) {
            int j = threadIdx.x + k * BT;
            uu[k] = j < deg ? (a.ckey ? a.ckey[beg + j] : a.col[beg + j]) : -1;
            ww[k] = (j < deg && !UNIT) ? (VT)a.w[beg + j] : (VT)1;
        }
        for (int r0 = 0; r0 < deg; r0 += BT * E) {          // block-uniform rounds
            int cc[E];
            if (r0 > 0 && !GALA_BLOCK_PIPE) {
#pragma unroll
                for (int k = 0; k < E; ++k) {
                    int j = r0 + threadIdx.x + k * BT;
                    uu[k] = j < deg ? (a.ckey ? a.ckey[beg + j] : a.col[beg + j]) : -1;
                    ww[k] = (j < deg && !UNIT) ? (VT)a.w[beg + j] : (VT)1;
                }
            }
            // next round's entries in flight during this round's gathers and inserts
            int nu[E];
            VT nw[E];
            if (GALA_BLOCK_PIPE) {
#pragma unroll
                for (int k = 0; k < E; ++k) {
                    int j = r0 + BT * E + threadIdx.x + k * BT;
                    nu[k] = j < deg ? (a.ckey ? a.ckey[beg + j] : a.col[beg + j]) : -1;
                    nw[k] = (j < deg && !UNIT) ? (VT)a.w[beg + j] : (VT)1;
                }
            }
            if (a.ckey) {
#pragma unroll
                for (int k = 0; k < E; ++k) cc[k] = uu[k];
            } else {
#pragma unroll
                for (int k = 0; k < E; ++k) cc[k] = (uu[k] >= 0 && uu[k] != v) ? a.C[uu[k]] : -1;
            }
#pragma unroll
            for (int k = 0; k < E; ++k)
                if (cc[k] == cv) { own += (long long)ww[k]; cc[k] = -1; }
#pragma unroll
            for (int k = 0; k < E; ++k) {
                const unsigned peers = __match_any_sync(FULLMASK, cc[k] >= 0 ? cc[k] : -1 - lane);
                const VT sum = UNIT ? (VT)__popc(peers) : group_sum(peers, cc[k] >= 0 ? ww[k] : (VT)0, s_scr[wib]);
                bool gfresh = false;
                int gslot = -1;
                if (cc[k] >= 0 && lane == __ffs(peers) - 1) {
                    bool fresh;
                    int slot = -1;
                    unsigned g0 = hash_slot2(cc[k], gmask);
                    // (the short-row class's arena never spills and its grid can exceed the H1 tables)
                    const int tmode = CLS == 1 ? 0 : a.table_mode;
                    if (tmode == 0) {                 // hierarchical: H0 first (own hash), H1 on collision
                        slot = ht_insert4<VT, true>(cc[k], sum, keys, vals, smask, hash_slot(cc[k], smask), win, &fresh);
                    } else if (tmode == 2) {          // unified: one hash over the s + g buckets
                        const unsigned uh = (unsigned)(((unsigned long long)(unsigned)cc[k] * 2654435761ull) %
                                                       (unsigned long long)(tcap + gc));
                        if (uh < (unsigned)tcap) slot = ht_insert4<VT, true>(cc[k], sum, keys, vals, smask, uh, win, &fresh);
                        else g0 = uh - (unsigned)tcap;
                    }                                 // global-only: H1 always
                    if (slot < 0) {
                        gslot = ht_insert4<ull, false>(cc[k], (ull)sum, gkeys, gvals, gmask, g0, (int)gc, &gfresh);
                        ++my_h1;
                    } else {
                        ++my_h0;
                    }
                }
                if (__any_sync(FULLMASK, gfresh)) append_fresh<int>(gfresh, gslot, FULLMASK, &s_gcnt, glist);
            }
            if (GALA_BLOCK_PIPE) {
#pragma unroll
                for (int k = 0; k < E; ++k) { uu[k] = nu[k]; ww[k] = nw[k]; }
            }
        }
        __syncthreads();
        const int gm = s_gcnt;
        const long long dv = q.dv;
        A best;
        best.init(a.idbits, a.idmask);
        my_k += (threadIdx.x == 0) ? (unsigned)gm : 0u;
        my_k1 += (threadIdx.x == 0) ? (ull)gm : 0ull;
        // evaluate and clear the used H0 prefix, four slots (one 16-byte key load) per thread
        // (two groups per pass measured slower: the extra registers halve the resident blocks)
        for (int t0 = threadIdx.x * 4; t0 < tcap; t0 += BT * 4) {
            const int4 k4 = *reinterpret_cast<const int4*>(keys + t0);
            const int cs[4] = {k4.x, k4.y, k4.z, k4.w};
            if ((k4.x & k4.y & k4.z & k4.w) == -1) continue;   // all four empty
            long long ws[4], sg[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                ws[k] = cs[k] >= 0 ? (long long)vals[t0 + k] : 0;
                sg[k] = cs[k] >= 0 ? a.Sig[cs[k]] : 0;
            }
            *reinterpret_cast<int4*>(keys + t0) = make_int4(-1, -1, -1, -1);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                if (cs[k] < 0) continue;
                vals[t0 + k] = 0;
                ++my_k;
                ++my_k0;
                best.offer(gain<ST>(qW, p, ws[k], sg[k], dv), cs[k]);
            }
        }
        for (int t = threadIdx.x; t < gm; t += BT) {
            int slot = glist[t];
            int c = gkeys[slot];
            long long wc = (long long)gvals[slot];
            gkeys[slot] = -1;
            gvals[slot] = 0;
            best.offer(gain<ST>(qW, p, wc, a.Sig[c], dv), c);
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
        own = warp_sum_ll(own);
        if (lane == 0) { r_a[wib] = best; r_own[wib] = own; }
        __syncthreads();
        if (wib == 0) {
            if (lane < BT / 32) { best = r_a[lane]; own = r_own[lane]; }
            else { best.init(a.idbits, a.idmask); own = 0; }
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
            own = warp_sum_ll(own);
            if (lane == 0) {
                if (a.check && own != a.dp[v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
                a.nextC[v] = decide_final<ST>(cv, q.szv, dv, own, q.sigv, best, a.size, qW, p);
                my_k += own ? 1u : 0u;
                s_gcnt = 0;
            }
        }
        __syncthreads();   // table / list / s_item reuse
    }
    ull vals5[5] = {(ull)my_k, my_h0, my_h1, my_k0, my_k1};
    ull* const dsts5[5] = {&a.ctr->bin_k[bin], &a.ctr->h0_acc, &a.ctr->h1_acc, &a.ctr->h0_keys, &a.ctr->h1_keys};
    block_add_counters<BT, 5>(vals5, dsts5);
}

// ---------------------------------------------------------------------------
// a3/a4, first iteration of a level: every vertex is a singleton (C[u] = u,
// Sig[u] = d(u), size 1, d'(v) = 0) and rows hold distinct columns, so
// d_c(v) = w(v,u) for c = u and no aggregation is needed:
//   score(u) = qW w(v,u) - p d(u) d(v),  stay = 0,
//   move to the best u iff score > 0 and u < v (swap suppression, both
//   singletons) — the iteration-1 closed form.  G lanes per
//   vertex stream the row, 4 entries per lane in flight.
// ---------------------------------------------------------------------------
template <int G, int M, bool UNIT>
__device__ __forceinline__ unsigned decide_single_bin(QView queue, int bin, const DecideArgs& a,
                                                      typename ModeT<M>::ST qW, typename ModeT<M>::ST p) {
    typedef typename ModeT<M>::ST ST;
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const int gid = lane / G, gl = lane % G;
    const long long count = (long long)a.ctr->bin_count[bin];
    const long long nwarps = (long long)gridDim.x * (blockDim.x >> 5);
    const long long per = 32 / G;
    unsigned my_k = 0;
    for (long long base = ((long long)blockIdx.x * (blockDim.x >> 5) + wib) * per; base < count; base += nwarps * per) {
        const long long i = base + gid;
        const bool valid = i < count;
        QRec q;
        if (valid) q = queue[i];
        const int v = valid ? q.v : 0;
        const int64_t beg = valid ? q.beg : 0;
        const int deg = valid ? q.deg : 0;
        const long long dv = valid ? q.dv : 0;
        Arg<ST, ModeT<M>::PK> best;
        best.init(a.idbits, a.idmask);
        int dmax = deg;   // warp-uniform round count: max row length of the warp's groups
#pragma unroll
        for (int o = 16; o >= G; o >>= 1) dmax = max(dmax, __shfl_xor_sync(FULLMASK, dmax, o));
        for (int r0 = 0; r0 < dmax; r0 += 4 * G) {
            int uu[4];
            long long ww[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                int j = r0 + gl + t * G;
                uu[t] = j < deg ? a.col[beg + j] : -1;
                ww[t] = (j < deg && !UNIT) ? a.w[beg + j] : 1;
            }
            long long du[4];
#pragma unroll
            for (int t = 0; t < 4; ++t) du[t] = (uu[t] >= 0 && uu[t] != v) ? a.Sig[uu[t]] : 0;
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (uu[t] < 0 || uu[t] == v) continue;
                my_k++;
                best.offer(gain<ST>(qW, p, ww[t], du[t], dv), uu[t]);
            }
        }
#pragma unroll
        for (int off = G / 2; off > 0; off >>= 1) best.xor_merge(off);
        if (valid && gl == 0) {
            int tgt = v;
            if (best.valid() && best.score() > (ST)0 && best.comm() < v) tgt = best.comm();
            if (a.check && a.dp[v] != 0) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            a.nextC[v] = tgt;
        }
    }
    return my_k;
}

// first iteration: bins 0-3 in one launch (G ~ row length / 4), the other bins one launch each
template <int M, bool UNIT>
__global__ void __launch_bounds__(256, GALA_SINGLE_MINB) k_decide_single_small(QRec* queues, long long qstride,
                                                             DecideArgs a, typename ModeT<M>::ST qW,
                                                             typename ModeT<M>::ST p) {
    const unsigned kk[4] = {decide_single_bin<1, M, UNIT>(qview(queues, qstride, BIN_S4), BIN_S4, a, qW, p),
                            decide_single_bin<2, M, UNIT>(qview(queues, qstride, BIN_S8), BIN_S8, a, qW, p),
                            decide_single_bin<4, M, UNIT>(qview(queues, qstride, BIN_S16), BIN_S16, a, qW, p),
                            decide_single_bin<8, M, UNIT>(qview(queues, qstride, BIN_S32), BIN_S32, a, qW, p)};
#pragma unroll
    for (int b = 0; b < 4; ++b) {
        ull t = block_sum_ull<256>((ull)kk[b]);
        if (threadIdx.x == 0 && t) atomicAdd(&a.ctr->bin_k[b], t);
    }
}
template <int M, bool UNIT>
__global__ void __launch_bounds__(256, GALA_SINGLE_MINB) k_decide_single(QView queue, int bin, DecideArgs a,
                                                       typename ModeT<M>::ST qW, typename ModeT<M>::ST p) {
    ull t = block_sum_ull<256>((ull)decide_single_bin<32, M, UNIT>(queue, bin, a, qW, p));
    if (threadIdx.x == 0 && t) atomicAdd(&a.ctr->bin_k[bin], t);
}

// ---------------------------------------------------------------------------
// a4 (hubs, rows longer than the block bin): the hierarchical table of §4.2
// spread over the whole GPU.  A row is cut into HUB_CH-entry
// chunks; any block takes any chunk (dynamic cursor), sums it in a shared-
// memory table (one slot per distinct community of the chunk, never full) and
// flushes the distinct (c, w_c) pairs into the hub's global table (capacity a
// power of two >= 2 min(deg, n), load <= 1/2) -- the global level of the
// hierarchy.  Fresh global keys go to the hub's distinct list.  k_hub_eval
// then evaluates each hub's list with one block and clears the table, so the
// tables are empty between iterations.  Chunk ranges / table offsets of the
// queued hubs are laid out by k_hub_prep (one block).
// ---------------------------------------------------------------------------
#define HUB_CH 1024
#define HUB_BT 256
#define HUB_EV 2048
#define HUB_EVAL_BT 512
struct HubWork {
    int* keys;          // global tables (all hubs), -1 = empty
    ull* vals;
    int* list;          // distinct-slot lists
    long long* pref;    // [count+1] chunk prefix of the queued hubs
    long long* toff;    // [count+1] table offsets
    long long* loff;    // [count+1] list offsets
    long long* spref;   // [count+1] evaluation-slice prefix
    int* cnt;           // [count] distinct keys inserted (zero between iterations)
    long long* own;     // [count] d'(v) aggregated on the fly (zero between iterations)
    void* part;         // per evaluation slice: partial argmax (Arg of the level's mode)
    long long nlev;     // vertices of the level (bound on distinct communities)
};

__device__ __forceinline__ unsigned hub_hash(int c, unsigned mask) {
    return (unsigned)(((unsigned long long)(unsigned)c * 0x9E3779B97F4A7C15ull) >> 32) & mask;
}
__device__ __forceinline__ long long hub_cap(long long deg, long long nlev) {
    long long d = deg < nlev ? deg : nlev, c = 64;
    while (c < 2 * d) c <<= 1;
    return c;
}

// block-wide exclusive scan of NV int64 values per thread (1024 threads), carried over tiles
template <int NV>
struct TileScan {
    long long w[NV][32];
    long long carry[NV];
};
template <int NV>
__device__ __forceinline__ void tile_scan(TileScan<NV>& sh, const long long (&x)[NV], long long (&ex)[NV]) {
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    long long inc[NV];
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        inc[k] = x[k];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            long long y = __shfl_up_sync(FULLMASK, inc[k], o);
            if (lane >= o) inc[k] += y;
        }
        if (lane == 31) sh.w[k][wib] = inc[k];
    }
    __syncthreads();
    if (wib == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            long long v = sh.w[k][lane], iv = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                long long y = __shfl_up_sync(FULLMASK, iv, o);
                if (lane >= o) iv += y;
            }
            sh.w[k][lane] = iv - v;
        }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < NV; ++k) ex[k] = sh.carry[k] + sh.w[k][wib] + inc[k] - x[k];
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1)
#pragma unroll
        for (int k = 0; k < NV; ++k) sh.carry[k] = ex[k] + x[k];
    __syncthreads();
}

// exclusive scans of (chunks, table capacity, list length) over the queued hubs
__global__ void __launch_bounds__(1024) k_hub_prep(QView queue, const IterCounters* __restrict__ ctr, HubWork h) {
    __shared__ TileScan<3> sh;
    const long long count = (long long)ctr->bin_count[BIN_HUB];
    if (threadIdx.x < 3) sh.carry[threadIdx.x] = 0;
    __syncthreads();
    for (long long t0 = 0; t0 < count; t0 += 1024) {
        const long long i = t0 + threadIdx.x;
        long long x[3] = {0, 0, 0}, ex[3];
        if (i < count) {
            const long long deg = queue[i].deg;
            x[0] = (deg + HUB_CH - 1) / HUB_CH;
            x[1] = hub_cap(deg, h.nlev);
            x[2] = deg < h.nlev ? deg : h.nlev;
        }
        tile_scan<3>(sh, x, ex);
        if (i < count) { h.pref[i] = ex[0]; h.toff[i] = ex[1]; h.loff[i] = ex[2]; }
    }
    if (threadIdx.x == 0) { h.pref[count] = sh.carry[0]; h.toff[count] = sh.carry[1]; h.loff[count] = sh.carry[2]; }
}

// last i in [0, count) with pref[i] <= item
__device__ __forceinline__ long long hub_find(const long long* __restrict__ pref, long long count, long long item) {
    long long lo = 0, hi = count - 1;
    while (lo < hi) {
        long long mid = (lo + hi + 1) >> 1;
        if (pref[mid] <= item) lo = mid; else hi = mid - 1;
    }
    return lo;
}

template <int M, bool UNIT>
__global__ void __launch_bounds__(HUB_BT) k_hub_agg(QView queue, DecideArgs a, HubWork h) {
    typedef typename ModeT<M>::VT VT;
    constexpr int SCAP = 2 * HUB_CH;
    constexpr int E = HUB_CH / HUB_BT;
    __shared__ int keys[SCAP];
    __shared__ VT vals[SCAP];
    __shared__ short list[HUB_CH];
    __shared__ VT s_scr[HUB_BT / 32][32];
    __shared__ long long s_item;
    __shared__ int s_cnt;
    if (a.ckey && !*a.ckey_valid) a.ckey = nullptr;
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    for (int j = threadIdx.x; j < SCAP; j += HUB_BT) { keys[j] = -1; vals[j] = 0; }
    if (threadIdx.x == 0) s_cnt = 0;
    const long long count = (long long)a.ctr->bin_count[BIN_HUB];
    if (count == 0) return;
    const long long total = h.pref[count];
    for (;;) {
        if (threadIdx.x == 0) s_item = (long long)atomicAdd(&a.ctr->cursor[BIN_HUB], 1ull);
        __syncthreads();
        const long long item = s_item;
        if (item >= total) break;
        const long long i = hub_find(h.pref, count, item);
        const QRec q = queue[i];
        const int v = q.v, cv = q.cv;
        const long long j0 = (item - h.pref[i]) * HUB_CH;
        int cc[E];
        VT ww[E];
#pragma unroll
        for (int k = 0; k < E; ++k) {
            const long long j = j0 + threadIdx.x + k * HUB_BT;
            int u = -1;
            if (j < q.deg) u = a.ckey ? a.ckey[q.beg + j] : a.col[q.beg + j];
            cc[k] = u;
            ww[k] = (j < q.deg && !UNIT) ? (VT)a.w[q.beg + j] : (VT)1;
        }
        if (!a.ckey) {
#pragma unroll
            for (int k = 0; k < E; ++k) cc[k] = (cc[k] >= 0 && cc[k] != v) ? a.C[cc[k]] : -1;
        }
        // the own community only feeds d'(v): summed in registers, never inserted
        long long own = 0;
#pragma unroll
        for (int k = 0; k < E; ++k)
            if (cc[k] == cv) { own += (long long)ww[k]; cc[k] = -1; }
#pragma unroll
        for (int k = 0; k < E; ++k) {
            const unsigned peers = __match_any_sync(FULLMASK, cc[k] >= 0 ? cc[k] : -1 - lane);
            const VT sum = UNIT ? (VT)__popc(peers) : group_sum(peers, cc[k] >= 0 ? ww[k] : (VT)0, s_scr[wib]);
            bool fresh = false;
            int slot = -1;
            if (cc[k] >= 0 && lane == __ffs(peers) - 1)
                slot = ht_insert4<VT, true>(cc[k], sum, keys, vals, SCAP - 1, hash_slot(cc[k], SCAP - 1), SCAP, &fresh);
            append_fresh<short>(fresh, slot, FULLMASK, &s_cnt, list);
        }
        own = warp_sum_ll(own);
        if (lane == 0 && own) atomicAdd(reinterpret_cast<ull*>(&h.own[i]), (ull)own);
        __syncthreads();
        const int m = s_cnt;
        const long long toff = h.toff[i], cap = h.toff[i + 1] - toff, loff = h.loff[i];
        int* gk = h.keys + toff;
        ull* gv = h.vals + toff;
        const unsigned gmask = (unsigned)(cap - 1);
        for (int t0 = threadIdx.x & ~31; t0 < m; t0 += HUB_BT) {   // warp-uniform trips
            const int t = t0 + lane;
            bool fresh = false;
            int gs = -1;
            if (t < m) {
                const int slot = list[t];
                const int c = keys[slot];
                const ull wv = (ull)vals[slot];
                keys[slot] = -1;
                vals[slot] = 0;
                gs = ht_insert<ull>(c, wv, gk, gv, gmask, hub_hash(c, gmask), (int)min(cap, (long long)INT_MAX), &fresh);
            }
            // one list-counter atomic per warp instead of one per fresh key
            const unsigned fm = __ballot_sync(FULLMASK, fresh);
            if (fm) {
                const int lead = __ffs(fm) - 1;
                int base = 0;
                if (lane == lead) base = atomicAdd(&h.cnt[i], __popc(fm));
                base = __shfl_sync(FULLMASK, base, lead);
                if (fresh) h.list[loff + base + __popc(fm & lanemask_lt())] = gs;
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) s_cnt = 0;
    }
}

// evaluation slices per hub (at least one, so every hub gets a partial)
__global__ void __launch_bounds__(1024) k_hub_prep2(const IterCounters* __restrict__ ctr, HubWork h) {
    __shared__ TileScan<1> sh;
    const long long count = (long long)ctr->bin_count[BIN_HUB];
    if (threadIdx.x == 0) sh.carry[0] = 0;
    __syncthreads();
    for (long long t0 = 0; t0 < count; t0 += 1024) {
        const long long i = t0 + threadIdx.x;
        long long x[1] = {0}, ex[1];
        if (i < count) x[0] = h.cnt[i] > HUB_EV ? (h.cnt[i] + HUB_EV - 1) / HUB_EV : 1;
        tile_scan<1>(sh, x, ex);
        if (i < count) h.spref[i] = ex[0];
    }
    if (threadIdx.x == 0) h.spref[count] = sh.carry[0];
}

// slice (hub i, entries [s HUB_EV, (s+1) HUB_EV) of its list): gains, partial argmax, clear slots
template <int M, bool UNIT>
__global__ void __launch_bounds__(HUB_EVAL_BT) k_hub_eval(QView queue, DecideArgs a, HubWork h,
                                                          typename ModeT<M>::ST qW, typename ModeT<M>::ST p) {
    typedef typename ModeT<M>::ST ST;
    typedef Arg<ST, ModeT<M>::PK> A;
    __shared__ A r_a[HUB_EVAL_BT / 32];
    __shared__ long long s_item;
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const long long count = (long long)a.ctr->bin_count[BIN_HUB];
    if (count == 0) return;
    const long long total = h.spref[count];
    A* part = reinterpret_cast<A*>(h.part);
    for (;;) {
        if (threadIdx.x == 0) s_item = (long long)atomicAdd(&a.ctr->cursor2, 1ull);
        __syncthreads();
        const long long item = s_item;
        if (item >= total) break;
        const long long i = hub_find(h.spref, count, item);
        const int cv = queue[i].cv;
        const long long dv = queue[i].dv;
        const long long t0 = (item - h.spref[i]) * HUB_EV;
        const long long t1 = min(t0 + HUB_EV, (long long)h.cnt[i]);
        const long long toff = h.toff[i], loff = h.loff[i];
        A best;
        best.init(a.idbits, a.idmask);
        // the slice's list entries, then their slots, then Sigma_tot of their communities, each
        // batch issued before any use: three dependent load rounds per thread, not three per entry
        constexpr int U = HUB_EV / HUB_EVAL_BT;
        long long slot[U];
        int c[U];
        long long wc[U], sg[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
            const long long t = t0 + threadIdx.x + (long long)k * HUB_EVAL_BT;
            slot[k] = t < t1 ? toff + h.list[loff + t] : -1;
        }
#pragma unroll
        for (int k = 0; k < U; ++k) {
            c[k] = slot[k] >= 0 ? h.keys[slot[k]] : -1;
            wc[k] = slot[k] >= 0 ? (long long)h.vals[slot[k]] : 0;
        }
#pragma unroll
        for (int k = 0; k < U; ++k) sg[k] = (c[k] >= 0 && c[k] != cv) ? a.Sig[c[k]] : 0;
#pragma unroll
        for (int k = 0; k < U; ++k) {
            if (slot[k] < 0) continue;
            h.keys[slot[k]] = -1;
            h.vals[slot[k]] = 0;
            if (c[k] != cv) best.offer(gain<ST>(qW, p, wc[k], sg[k], dv), c[k]);
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
        if (lane == 0) r_a[wib] = best;
        __syncthreads();
        if (wib == 0) {
            if (lane < HUB_EVAL_BT / 32) best = r_a[lane];
            else best.init(a.idbits, a.idmask);
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
            if (lane == 0) part[item] = best;
        }
        __syncthreads();
    }
}

// one warp per hub: merge its slices' partials, decide, reset the hub's counters
template <int M, bool UNIT>
__global__ void __launch_bounds__(256) k_hub_final(QView queue, DecideArgs a, HubWork h, typename ModeT<M>::ST qW,
                                                   typename ModeT<M>::ST p) {
    typedef typename ModeT<M>::ST ST;
    typedef Arg<ST, ModeT<M>::PK> A;
    const int lane = lane_id();
    const long long count = (long long)a.ctr->bin_count[BIN_HUB];
    const A* part = reinterpret_cast<const A*>(h.part);
    unsigned my_k = 0;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long i = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < count; i += nw) {
        A best;
        best.init(a.idbits, a.idmask);
        for (long long s = h.spref[i] + lane; s < h.spref[i + 1]; s += 32) {
            A o = part[s];
            if (o.valid()) best.offer(o.score(), o.comm());
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
        if (lane == 0) {
            const QRec q = queue[i];
            const long long own = h.own[i];
            if (a.check && own != a.dp[q.v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            a.nextC[q.v] = decide_final<ST>(q.cv, q.szv, q.dv, own, q.sigv, best, a.size, qW, p);
            my_k += (unsigned)h.cnt[i] + (own ? 1u : 0u);
            h.cnt[i] = 0;
            h.own[i] = 0;
        }
    }
    ull k = block_sum_ull<256>((ull)my_k);
    if (threadIdx.x == 0 && k) atomicAdd(&a.ctr->bin_k[BIN_HUB], k);
}

// First iteration of a level (all singletons, rows with distinct columns): a hub needs no
// aggregation at all -- score(u) = qW w(v,u) - p d(u) d(v) per entry (decide_single_bin's closed
// form).  Any block takes any HUB_CH-entry chunk of any hub (prefix h.pref from k_hub_prep) and
// writes the chunk's partial argmax; k_hub_single_final merges them per hub.
template <int M, bool UNIT>
__global__ void __launch_bounds__(HUB_BT) k_hub_single_chunk(QView queue, DecideArgs a, HubWork h,
                                                             typename ModeT<M>::ST qW, typename ModeT<M>::ST p) {
    typedef typename ModeT<M>::ST ST;
    typedef Arg<ST, ModeT<M>::PK> A;
    constexpr int E = HUB_CH / HUB_BT;
    __shared__ A r_a[HUB_BT / 32];
    __shared__ long long s_item;
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    const long long count = (long long)a.ctr->bin_count[BIN_HUB];
    if (count == 0) return;
    const long long total = h.pref[count];
    A* part = reinterpret_cast<A*>(h.part);
    for (;;) {
        if (threadIdx.x == 0) s_item = (long long)atomicAdd(&a.ctr->cursor[BIN_HUB], 1ull);
        __syncthreads();
        const long long item = s_item;
        if (item >= total) break;
        const long long i = hub_find(h.pref, count, item);
        const QRec q = queue[i];
        const long long j0 = (item - h.pref[i]) * HUB_CH;
        int uu[E];
        long long ww[E], du[E];
#pragma unroll
        for (int k = 0; k < E; ++k) {
            const long long j = j0 + threadIdx.x + k * HUB_BT;
            uu[k] = j < q.deg ? a.col[q.beg + j] : -1;
            ww[k] = (j < q.deg && !UNIT) ? a.w[q.beg + j] : 1;
        }
#pragma unroll
        for (int k = 0; k < E; ++k) du[k] = (uu[k] >= 0 && uu[k] != q.v) ? a.Sig[uu[k]] : 0;
        A best;
        best.init(a.idbits, a.idmask);
#pragma unroll
        for (int k = 0; k < E; ++k)
            if (uu[k] >= 0 && uu[k] != q.v) best.offer(gain<ST>(qW, p, ww[k], du[k], q.dv), uu[k]);
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
        if (lane == 0) r_a[wib] = best;
        __syncthreads();
        if (wib == 0) {
            if (lane < HUB_BT / 32) best = r_a[lane];
            else best.init(a.idbits, a.idmask);
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
            if (lane == 0) part[item] = best;
        }
        __syncthreads();
    }
}

template <int M, bool UNIT>
__global__ void __launch_bounds__(256) k_hub_single_final(QView queue, DecideArgs a, HubWork h) {
    typedef typename ModeT<M>::ST ST;
    typedef Arg<ST, ModeT<M>::PK> A;
    const int lane = lane_id();
    const long long count = (long long)a.ctr->bin_count[BIN_HUB];
    const A* part = reinterpret_cast<const A*>(h.part);
    ull my_k = 0;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long i = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < count; i += nw) {
        A best;
        best.init(a.idbits, a.idmask);
        for (long long s = h.pref[i] + lane; s < h.pref[i + 1]; s += 32) {
            A o = part[s];
            if (o.valid()) best.offer(o.score(), o.comm());
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
        if (lane == 0) {
            const QRec q = queue[i];
            int tgt = q.v;
            if (best.valid() && best.score() > (ST)0 && best.comm() < q.v) tgt = best.comm();
            if (a.check && a.dp[q.v] != 0) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            a.nextC[q.v] = tgt;
            my_k += (ull)q.deg;
        }
    }
    ull k = block_sum_ull<256>(my_k);
    if (threadIdx.x == 0 && k) atomicAdd(&a.ctr->bin_k[BIN_HUB], k);
}

// per level: number of rows longer than t, and the table / list space they can need
__global__ void k_hub_size(long long n, const int64_t* __restrict__ rp, long long t, long long nlev,
                           ull* __restrict__ out) {
    ull c = 0, cap = 0, dist = 0;
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
        const long long deg = rp[v + 1] - rp[v];
        if (deg > t) { c++; cap += (ull)hub_cap(deg, nlev); dist += (ull)(deg < nlev ? deg : nlev); }
    }
    if (c) {
        atomicAdd(&out[0], c);
        atomicAdd(&out[1], cap);
        atomicAdd(&out[2], dist);
    }
}

// ---------------------------------------------------------------------------
// a4, hubs (rows longer than the block bin) on a THREAD-BLOCK CLUSTER: the hierarchical
// table's upper level (§4.2: "if H0 cannot hold a community, H1") lives in the
// distributed shared memory of CS CTAs instead of global memory.  One cluster per hub vertex
// (dynamic fetch by CTA 0, broadcast over DSMEM):
//   * every CTA streams a contiguous 1/CS of the row (E entries per thread in flight), combines
//     the equal communities of each 32-entry chunk with __match_any_sync (Alg. 2) and inserts the
//     chunk's distinct (c, sum) into the table of the OWNER CTA of c (hub_hash bits), a packed
//     64-bit slot per key (kv_insert through the cluster-mapped address: DSMEM atomics);
//   * the own community only feeds d'(v) (summed in registers, one DSMEM add per CTA);
//   * cluster barrier; each CTA evaluates and clears the occupied slots of its own table
//     (Sigma_tot gathered once per distinct community), block argmax, partial written into
//     CTA 0 over DSMEM; cluster barrier; CTA 0 decides (reading c1/c4/c5).
// Table: nextpow2(2 min(deg, n_level)) slots split evenly over the CS CTAs (load <= 1/2, never
// spills); used on levels whose longest row fits CS * CL_SLOTS slots and whose aggregates are
// 32-bit (not DM_W128), else the global multi-block hub path above runs.
// ---------------------------------------------------------------------------
#include <cooperative_groups.h>
#define CL_CS 8          // CTAs per cluster (portable maximum)
#define CL_SLOTS 16384   // packed slots per CTA (128 KB of shared memory)
#define CL_BT 512
#define CL_E 4
template <int M, bool UNIT>
__global__ void __cluster_dims__(CL_CS, 1, 1) __launch_bounds__(CL_BT, 1)
    k_decide_cluster(QView queue, DecideArgs a, typename ModeT<M>::ST qW, typename ModeT<M>::ST p) {
    namespace cg = cooperative_groups;
    typedef typename ModeT<M>::ST ST;
    typedef Arg<ST, ModeT<M>::PK> A;
    static_assert(sizeof(typename ModeT<M>::VT) == 4, "packed slots need 32-bit aggregates");
    cg::cluster_group cl = cg::this_cluster();
    const unsigned crank = cl.block_rank();
    extern __shared__ __align__(16) ull ctbl[];
    // hub index and own-community sum double-buffered by hub parity: two cluster barriers per hub
    // (the next hub's index is fetched before the barrier that publishes the partials)
    __shared__ long long s_item[2];
    __shared__ long long s_own[2];
    __shared__ A s_part[CL_CS];
    __shared__ A r_a[CL_BT / 32];
    __shared__ unsigned s_scr[CL_BT / 32][32];
    if (a.ckey && !*a.ckey_valid) a.ckey = nullptr;
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    for (int j = threadIdx.x; j < CL_SLOTS; j += CL_BT) ctbl[j] = KV_EMPTY;
    if (threadIdx.x == 0) { s_own[0] = 0; s_own[1] = 0; }
    const long long count = (long long)a.ctr->bin_count[BIN_HUB];
    ull* const cursor = &a.ctr->cursor[BIN_HUB];
    long long* const own0 = cl.map_shared_rank(s_own, 0);
    A* const part0 = cl.map_shared_rank(s_part, 0);
    const long long* const item0 = cl.map_shared_rank(s_item, 0);
    unsigned my_k = 0;
    if (crank == 0 && threadIdx.x == 0) s_item[0] = (long long)atomicAdd(cursor, 1ull);
    cl.sync();   // tables initialised everywhere, the first hub index published
    for (int par = 0;; par ^= 1) {
        const long long i = item0[par];
        if (i >= count) {   // no CTA may exit while another still reads its shared memory (s_item)
            cl.sync();
            break;
        }
        const QRec q = queue[i];
        const int v = q.v, deg = q.deg, cv = q.cv;
        const long long span = deg < a.nlev ? deg : a.nlev;
        long long need = 64LL * CL_CS;
        while (need < 2 * span) need <<= 1;
        const unsigned tmask = (unsigned)(need / CL_CS) - 1;   // this hub's slots per CTA
        const long long per = (deg + CL_CS - 1) / CL_CS;
        const long long r0 = (long long)crank * per, r1 = min((long long)deg, r0 + per);
        long long own = 0;
        for (long long j0 = r0; j0 < r1; j0 += (long long)CL_BT * CL_E) {   // block-uniform rounds
            int cc[CL_E];
            unsigned ww[CL_E];
#pragma unroll
            for (int k = 0; k < CL_E; ++k) {
                const long long j = j0 + threadIdx.x + (long long)k * CL_BT;
                const bool in = j < r1;
                int u = in ? (a.ckey ? a.ckey[q.beg + j] : a.col[q.beg + j]) : -1;
                ww[k] = (in && !UNIT) ? (unsigned)a.w[q.beg + j] : 1u;
                if (!a.ckey) u = (u >= 0 && u != v) ? a.C[u] : -1;
                cc[k] = in ? u : -1;
            }
#pragma unroll
            for (int k = 0; k < CL_E; ++k) {
                if (cc[k] == cv) { own += (long long)ww[k]; cc[k] = -1; }
                const unsigned peers = __match_any_sync(FULLMASK, cc[k] >= 0 ? cc[k] : -1 - lane);
                const unsigned sum = UNIT ? (unsigned)__popc(peers) : group_sum(peers, cc[k] >= 0 ? ww[k] : 0u, s_scr[wib]);
                if (cc[k] >= 0 && lane == __ffs(peers) - 1) {
                    const unsigned hh = hub_hash(cc[k], 0xFFFFFFFFu);
                    ull* const t = cl.map_shared_rank(ctbl, hh % CL_CS);
                    bool fresh;
                    kv_insert(cc[k], sum, t, tmask, (hh / CL_CS) & tmask, (int)tmask + 1, &fresh);
                }
            }
        }
        own = warp_sum_ll(own);
        if (lane == 0 && own) atomicAdd(reinterpret_cast<ull*>(own0 + par), (ull)own);
        cl.sync();   // every insert (and every own contribution) has landed
        const long long dv = q.dv;
        A best;
        best.init(a.idbits, a.idmask);
        for (unsigned t0 = threadIdx.x * 2; t0 <= tmask; t0 += CL_BT * 2) {   // two slots (16 bytes) per load
            const ulonglong2 kv = *reinterpret_cast<const ulonglong2*>(ctbl + t0);
            const ull e[2] = {kv.x, kv.y};
            if (e[0] == KV_EMPTY && e[1] == KV_EMPTY) continue;
            long long sg[2];
#pragma unroll
            for (int k = 0; k < 2; ++k) sg[k] = e[k] != KV_EMPTY ? a.Sig[(int)(e[k] >> 32)] : 0;
            *reinterpret_cast<ulonglong2*>(ctbl + t0) = make_ulonglong2(KV_EMPTY, KV_EMPTY);
#pragma unroll
            for (int k = 0; k < 2; ++k) {
                if (e[k] == KV_EMPTY) continue;
                ++my_k;
                best.offer(gain<ST>(qW, p, (long long)(unsigned)e[k], sg[k], dv), (int)(e[k] >> 32));
            }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
        if (lane == 0) r_a[wib] = best;
        __syncthreads();
        if (wib == 0) {
            best = lane < CL_BT / 32 ? r_a[lane] : best;
            if (lane >= CL_BT / 32) best.init(a.idbits, a.idmask);
#pragma unroll
            for (int off = 16; off > 0; off >>= 1) best.xor_merge(off);
            if (lane == 0) part0[crank] = best;
        }
        if (crank == 0 && threadIdx.x == 0) s_item[par ^ 1] = (long long)atomicAdd(cursor, 1ull);   // next hub
        cl.sync();   // every CTA's partial is in CTA 0, the next hub index is published, tables clear
        if (crank == 0 && threadIdx.x == 0) {
            A b = s_part[0];
            for (int r = 1; r < CL_CS; ++r)
                if (s_part[r].valid()) b.offer(s_part[r].score(), s_part[r].comm());
            const long long ownv = s_own[par];
            if (a.check && ownv != a.dp[v]) atomicAdd(&a.ctr->dp_mismatch, 1ull);
            a.nextC[v] = decide_final<ST>(cv, q.szv, dv, ownv, q.sigv, b, a.size, qW, p);
            my_k += ownv ? 1u : 0u;
            s_own[par] = 0;   // reused two hubs later, after two more barriers
        }
    }
    ull k = block_sum_ull<CL_BT>((ull)my_k);
    if (threadIdx.x == 0 && k) atomicAdd(&a.ctr->bin_k[BIN_HUB], k);
}
