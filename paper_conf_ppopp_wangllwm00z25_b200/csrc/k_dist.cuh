// k_dist.cuh — kernels of the multi-GPU driver (§4.3).
// Rank r owns vertices [v0, v1); its graph is a "global-row" CSR (n rows, rows
// outside [v0, v1) empty, column ids global).  Community state (C, Sigma_tot,
// size, d) is replicated and updated identically on every rank from the
// global list of moves of the iteration.
#pragma once
#include "common.cuh"

// local row_ptr (n_own + 1, starting at 0) -> global-row row_ptr (n + 1)
__global__ void k_expand_rp(long long n, long long v0, long long v1, const int64_t* __restrict__ lrp,
                            int64_t* __restrict__ rp) {
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v <= n; v += (long long)gridDim.x * blockDim.x)
        rp[v] = v <= v0 ? 0 : (v >= v1 ? lrp[v1 - v0] : lrp[v - v0]);
}

// owned queued vertices whose decision differs -> local move list (v, new), block-aggregated
__global__ void __launch_bounds__(256) k_collect_moves(const IterCounters* __restrict__ ctr,
                                                       QRec* queues, long long qstride,
                                                       const int32_t* __restrict__ nextC, int2* __restrict__ moves,
                                                       ull* __restrict__ nmoves) {
    __shared__ unsigned s_cnt;
    __shared__ ull s_base;
    long long cnt[NBINS];
    long long total = 0;
#pragma unroll
    for (int b = 0; b < NBINS; ++b) { cnt[b] = (long long)ctr->bin_count[b]; total += cnt[b]; }
    for (long long t0 = (long long)blockIdx.x * 256; t0 < total; t0 += (long long)gridDim.x * 256) {
        const long long i = t0 + threadIdx.x;
        bool mover = false;
        int v = 0, nc = 0;
        if (i < total) {
            int b = 0;
            long long r = i;
#pragma unroll
            for (int k = 0; k < NBINS - 1; ++k)
                if (b == k && r >= cnt[k]) { r -= cnt[k]; b = k + 1; }
            const QRec q = qview(queues, qstride, b)[r];
            v = q.v;
            nc = nextC[v];
            mover = nc != q.cv;
        }
        if (threadIdx.x == 0) s_cnt = 0;
        __syncthreads();
        const unsigned m = __ballot_sync(FULLMASK, mover);
        unsigned off = 0;
        if (m && lane_id() == __ffs(m) - 1) off = atomicAdd(&s_cnt, (unsigned)__popc(m));
        off = __shfl_sync(FULLMASK, off, m ? __ffs(m) - 1 : 0) + __popc(m & lanemask_lt());
        __syncthreads();
        if (threadIdx.x == 0) s_base = s_cnt ? atomicAdd(nmoves, (ull)s_cnt) : 0;
        __syncthreads();
        if (mover) moves[s_base + off] = make_int2(v, nc);
    }
}

// dense exchange: this rank's slice of the next label array = C, then the local moves
__global__ void k_copy_range(long long v0, long long v1, const int32_t* __restrict__ src, int32_t* __restrict__ dst) {
    for (long long v = v0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += (long long)gridDim.x * blockDim.x)
        dst[v] = src[v];
}
__global__ void k_scatter_moves(const int2* __restrict__ moves, const ull* __restrict__ nmoves, int32_t* __restrict__ newC) {
    const long long m = (long long)*nmoves;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x)
        newC[moves[i].x] = moves[i].y;
}

// dense exchange: global move list = vertices whose gathered label differs, block-aggregated
__global__ void __launch_bounds__(256) k_diff_moves(int n, const int32_t* __restrict__ C,
                                                    const int32_t* __restrict__ newC, int2* __restrict__ moves,
                                                    ull* __restrict__ nmoves) {
    __shared__ unsigned s_cnt;
    __shared__ ull s_base;
    for (long long t0 = (long long)blockIdx.x * 256; t0 < n; t0 += (long long)gridDim.x * 256) {
        const long long v = t0 + threadIdx.x;
        const bool mover = v < n && newC[v] != C[v];
        if (threadIdx.x == 0) s_cnt = 0;
        __syncthreads();
        const unsigned m = __ballot_sync(FULLMASK, mover);
        unsigned off = 0;
        if (m && lane_id() == __ffs(m) - 1) off = atomicAdd(&s_cnt, (unsigned)__popc(m));
        off = __shfl_sync(FULLMASK, off, m ? __ffs(m) - 1 : 0) + __popc(m & lanemask_lt());
        __syncthreads();
        if (threadIdx.x == 0) s_base = s_cnt ? atomicAdd(nmoves, (ull)s_cnt) : 0;
        __syncthreads();
        if (mover) moves[s_base + off] = make_int2((int)v, newC[v]);
    }
}

// apply the global move list to the replicated state (identical on every rank):
// Sigma_tot / size by int atomics (order-independent), C <- new, stamp
__global__ void k_apply_list(const int2* __restrict__ moves, long long m, int32_t* __restrict__ C,
                             int64_t* __restrict__ Sig, int32_t* __restrict__ size, const int64_t* __restrict__ d,
                             int32_t* __restrict__ stamp, const Carry* __restrict__ carry,
                             IterCounters* __restrict__ ctr) {
    const int iter_id = carry->iter;
    if (blockIdx.x == 0 && threadIdx.x == 0) ctr->n_moved = (ull)m;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x) {
        const int v = moves[i].x, nc = moves[i].y;
        const int oc = C[v];
        const long long dv = d[v];
        C[v] = nc;
        stamp[v] = iter_id;
        atomicAdd(reinterpret_cast<ull*>(&Sig[oc]), (ull)(-dv));
        atomicAdd(reinterpret_cast<ull*>(&Sig[nc]), (ull)dv);
        atomicSub(&size[oc], 1);
        atomicAdd(&size[nc], 1);
    }
}

// counters to all-reduce: [sumDC, n_active, n_pruned, edges scanned, distinct communities]
__global__ void k_pack_counters(const Carry* __restrict__ carry, const IterCounters* __restrict__ ctr,
                                int64_t* __restrict__ vec) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    long long sd = 0, sk = 0;
    for (int b = 0; b < NBINS; ++b) { sd += (long long)ctr->bin_deg[b]; sk += (long long)ctr->bin_k[b]; }
    vec[0] = carry->sumDC;
    vec[1] = (long long)ctr->n_active;
    vec[2] = (long long)ctr->n_pruned;
    vec[3] = sd;
    vec[4] = sk;
}

// after the all-reduce: N' = qW sumDC - p S2, convergence (mode 1) exactly as k_reduce
__global__ void k_finish(const int64_t* __restrict__ vec, IterCounters* __restrict__ ctr, Carry* __restrict__ carry,
                         long long qW_hi, ull qW_lo, long long p, long long T_hi, ull T_lo, int mode) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const long long tdc = vec[0];
    const i128 S2 = mk128(carry->S2_hi, carry->S2_lo);
    const i128 Nn = mk128(qW_hi, qW_lo) * (i128)tdc - (i128)p * S2;
    const i128 N = mk128(carry->N_hi, carry->N_lo);
    int conv = 0;
    if (mode == 1) conv = (ctr->n_moved == 0) || (Nn - N < mk128(T_hi, T_lo));
    carry->N_prev_hi = hi128(N);
    carry->N_prev_lo = lo128(N);
    carry->N_hi = hi128(Nn);
    carry->N_lo = lo128(Nn);
    carry->sumDC = tdc;
    carry->converged = conv;
    carry->t_ns = globaltimer_ns();
    ctr->n_active = (ull)vec[1];
    ctr->n_pruned = (ull)vec[2];
    for (int b = 0; b < NBINS; ++b) { ctr->bin_deg[b] = 0; ctr->bin_k[b] = 0; }
    ctr->bin_deg[0] = (ull)vec[3];
    ctr->bin_k[0] = (ull)vec[4];
}

// partial coarse rows of all ranks (triplets) -> counting sort by row
__global__ void k_count_rows(long long m, const int32_t* __restrict__ row, long long* __restrict__ cnt) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x)
        atomicAdd(reinterpret_cast<ull*>(&cnt[row[i]]), 1ull);
}
__global__ void k_scatter_rows(long long m, const int32_t* __restrict__ row, const int32_t* __restrict__ col,
                               const int64_t* __restrict__ w, const long long* __restrict__ rp, long long* __restrict__ cur,
                               int32_t* __restrict__ orow, int32_t* __restrict__ ocol, int64_t* __restrict__ ow) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (long long)gridDim.x * blockDim.x) {
        const int r = row[i];
        const long long o = rp[r] + (long long)atomicAdd(reinterpret_cast<ull*>(&cur[r]), 1ull);
        orow[o] = r;
        ocol[o] = col[i];
        ow[o] = w[i];
    }
}

__global__ void k_iota(long long n, int32_t* __restrict__ x) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        x[i] = (int32_t)i;
}

// edge-balanced split of a CSR over `world` ranks: bounds[r] = smallest v with rp[v] >= r*nnz/world
__global__ void k_partition_bounds(long long n, const int64_t* __restrict__ rp, int world, long long* __restrict__ bounds) {
    const int r = threadIdx.x;
    if (r > world) return;
    if (r == 0) { bounds[0] = 0; return; }
    if (r == world) { bounds[world] = n; return; }
    const long long nnz = rp[n];
    const long long target = (long long)(((__int128)nnz * r + world - 1) / world);
    long long lo = 0, hi = n;
    while (lo < hi) {
        long long mid = (lo + hi) / 2;
        if (rp[mid] < target) lo = mid + 1; else hi = mid;
    }
    bounds[r] = lo;
}

// global-row CSR restricted to rows [lo, hi): rp'[v] = clamp(rp[v]) - rp[lo]
__global__ void k_restrict_rp(long long n, long long lo, long long hi, const int64_t* __restrict__ rp,
                              int64_t* __restrict__ out) {
    const int64_t a = rp[lo], b = rp[hi];
    for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v <= n; v += (long long)gridDim.x * blockDim.x) {
        int64_t x = rp[v];
        x = x < a ? a : (x > b ? b : x);
        out[v] = x - a;
    }
}

// partial coarse row lengths (send-to-owner phase 2): len[c] = rp[c + 1] - rp[c]
__global__ void k_row_lengths(long long k, const int64_t* __restrict__ rp, long long* __restrict__ len) {
    for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < k; c += (long long)gridDim.x * blockDim.x)
        len[c] = rp[c + 1] - rp[c];
}
