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
// ent[c'] += deg(v)
__global__ void k_coarsen_count(int n, const int64_t* __restrict__ rp, const int32_t* __restrict__ newid,
                                long long* __restrict__ ent) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x) {
        long long dg = rp[v + 1] - rp[v];
        if (dg) atomicAdd(reinterpret_cast<ull*>(&ent[newid[v]]), (ull)dg);
    }
}

// per-community hash capacity: nextpow2(2 * min(ent, k)), at least 2
__global__ void k_coarsen_cap(long long k, const long long* __restrict__ ent, long long* __restrict__ cap) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < k; c += (long long)gridDim.x * blockDim.x) {
        long long m = ent[c] < k ? ent[c] : k;
        long long x = 2;
        while (x < 2 * m) x <<= 1;
        cap[c] = ent[c] ? x : 0;
    }
}

// warp per vertex: insert (newid[u], w) into the table of newid[v].  Equal
// keys of a 32-entry chunk are combined first (__match_any_sync; popc on unit
// weights, shared-memory atomics onto the group leader otherwise) so the
// table sees one atomic per distinct key per chunk; the first inserter of a
// key bumps deg_new[c'].
template <bool UNIT>
__global__ void __launch_bounds__(256) k_coarsen_insert(int n, const int64_t* __restrict__ rp,
                                                        const int32_t* __restrict__ col,
                                                        const int64_t* __restrict__ w,
                                                        const int32_t* __restrict__ newid,
                                                        const long long* __restrict__ hoff, int* __restrict__ hkeys,
                                                        ull* __restrict__ hvals, long long* __restrict__ deg_new) {
    __shared__ ull s_acc[8][32];
    const int lane = lane_id(), wib = threadIdx.x >> 5;
    long long wid = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long v = wid; v < n; v += nw) {
        int cs = newid[v];
        int64_t b = rp[v], e = rp[v + 1];
        long long off = hoff[cs];
        unsigned mask = (unsigned)(hoff[cs + 1] - off) - 1u;
        int* keys = hkeys + off;
        ull* vals = hvals + off;
        for (int64_t j0 = b; j0 < e; j0 += 32) {
            int64_t j = j0 + lane;
            bool has = j < e;
            int key = has ? newid[col[j]] : (-1 - lane);
            ull wt = has ? (UNIT ? 1ull : (ull)w[j]) : 0ull;
            unsigned peers = __match_any_sync(FULLMASK, key);
            int leader = __ffs(peers) - 1;
            ull sum;
            if (UNIT) {
                sum = (ull)__popc(peers);
            } else {
                s_acc[wib][lane] = 0;
                __syncwarp();
                if (has) atomicAdd(&s_acc[wib][leader], wt);
                __syncwarp();
                sum = s_acc[wib][lane];
                __syncwarp();
            }
            if (has && lane == leader) {
                unsigned h = hash_slot(key, mask);
                for (;;) {
                    int k0 = *(volatile int*)&keys[h];
                    if (k0 == key) { atomicAdd(&vals[h], sum); break; }
                    if (k0 == -1) {
                        int old = atomicCAS(&keys[h], -1, key);
                        if (old == -1) {
                            atomicAdd(&vals[h], sum);
                            atomicAdd(reinterpret_cast<ull*>(&deg_new[cs]), 1ull);
                            break;
                        }
                        if (old == key) { atomicAdd(&vals[h], sum); break; }
                    }
                    h = (h + 1) & mask;
                }
            }
        }
    }
}

// largest c in [lo, hi] with hoff[c] <= t
__device__ __forceinline__ long long seg_search(const long long* __restrict__ hoff, long long lo, long long hi,
                                                long long t) {
    while (lo < hi) {
        long long mid = (lo + hi + 1) >> 1;
        if (hoff[mid] <= t) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// 256 consecutive table slots per block: the block's first/last slot find
// their community by binary search; every other slot searches only between
// the two (usually zero steps).  Occupied slots go to the coarse CSR rows.
__global__ void __launch_bounds__(256) k_coarsen_extract(long long k, long long total,
                                                         const long long* __restrict__ hoff,
                                                         const int* __restrict__ hkeys, const ull* __restrict__ hvals,
                                                         const long long* __restrict__ rp_new,
                                                         long long* __restrict__ fill, int32_t* __restrict__ col_new,
                                                         int64_t* __restrict__ w_new, int64_t* __restrict__ s_new) {
    __shared__ long long s_lo, s_hi;
    for (long long t0 = (long long)blockIdx.x * 256; t0 < total; t0 += (long long)gridDim.x * 256) {
        long long last = t0 + 255 < total ? t0 + 255 : total - 1;
        if (threadIdx.x == 0) s_lo = seg_search(hoff, 0, k - 1, t0);
        if (threadIdx.x == 32) s_hi = seg_search(hoff, 0, k - 1, last);
        __syncthreads();
        long long t = t0 + threadIdx.x;
        if (t < total) {
            int key = hkeys[t];
            if (key >= 0) {
                long long c = seg_search(hoff, s_lo, s_hi, t);
                ull pos = atomicAdd(reinterpret_cast<ull*>(&fill[c]), 1ull);
                long long o = rp_new[c] + (long long)pos;
                col_new[o] = key;
                w_new[o] = (int64_t)hvals[t];
                if (key == c) s_new[c] = (int64_t)hvals[t];
            }
        }
        __syncthreads();
    }
}

// coarse d(c') = Sigma_tot of the community (maintained exactly by phase 1)
__global__ void k_coarsen_deg(int n, const int32_t* __restrict__ C, const int32_t* __restrict__ minmem,
                              const int32_t* __restrict__ newid, const int64_t* __restrict__ Sig,
                              int64_t* __restrict__ d_new) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (long long)gridDim.x * blockDim.x)
        if (minmem[C[v]] == v) d_new[newid[v]] = Sig[C[v]];
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
