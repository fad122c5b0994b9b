// k_nmi.cuh — normalised mutual information of two partitions on the device (SURVEY.md §8(f)
// NEXT #4; Table 4 "NMI" against the LFR ground truth; definition of
// ref. [52], Strehl & Ghosh 2002):
//
//   NMI(X, Y) = I(X; Y) / sqrt(H(X) H(Y))
//   I(X; Y)   = sum_{a,b: n_ab > 0} (n_ab / n) ln(n n_ab / (n_a n_b))
//   H(X)      = -sum_{a: n_a > 0} (n_a / n) ln(n_a / n)
//
// Degenerate case (a side with one cluster, H = 0): 1 if both sides are single-cluster, else 0.
//
// Labels are int32 in [0, n).  Cluster sizes n_a, n_b are int32 histograms; the contingency
// counts n_ab live in a global open-addressing table keyed by the 64-bit pair (a << 32 | b)
// (CAS on the key, integer add on the count: exact and order-independent).  The three fp64
// sums are reduced in a fixed order (fixed grid, strided per thread, block tree, then the
// block partials in block order), so the result does not depend on scheduling.
#pragma once
#include "common.cuh"

#define NMI_BT 256
#define NMI_GRID 592   // 4 x 148 SMs: the partial-sum layout is fixed (deterministic order)
#define NMI_EMPTY 0xFFFFFFFFFFFFFFFFull

__global__ void __launch_bounds__(NMI_BT) k_nmi_count(long long n, const int32_t* __restrict__ x,
                                                      const int32_t* __restrict__ y, unsigned* __restrict__ na,
                                                      unsigned* __restrict__ nb, ull* __restrict__ keys,
                                                      unsigned* __restrict__ cnt, ull mask, int* __restrict__ bad) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        const int a = x[i], b = y[i];
        if (a < 0 || b < 0 || a >= n || b >= n) { *bad = 1; continue; }
        atomicAdd(&na[a], 1u);
        atomicAdd(&nb[b], 1u);
        const ull key = ((ull)(unsigned)a << 32) | (unsigned)b;
        ull h = (key * 0x9E3779B97F4A7C15ull) >> 17;
        for (;;) {   // linear probing; the table has >= 2n slots, so it never fills
            h &= mask;
            const ull k = keys[h];
            if (k == key) break;
            if (k == NMI_EMPTY) {
                const ull old = atomicCAS(&keys[h], NMI_EMPTY, key);
                if (old == NMI_EMPTY || old == key) break;
            }
            ++h;
        }
        atomicAdd(&cnt[h], 1u);
    }
}

__device__ __forceinline__ double nmi_block_sum(double v, double* s) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(FULLMASK, v, o);
    if ((threadIdx.x & 31) == 0) s[threadIdx.x >> 5] = v;
    __syncthreads();
    double t = 0;
    if (threadIdx.x == 0)
        for (int w = 0; w < NMI_BT / 32; ++w) t += s[w];
    __syncthreads();
    return t;
}

// partials[3 * block + {0, 1, 2}] = this block's share of I, H(X), H(Y)
__global__ void __launch_bounds__(NMI_BT) k_nmi_terms(long long n, const unsigned* __restrict__ na,
                                                      const unsigned* __restrict__ nb, const ull* __restrict__ keys,
                                                      const unsigned* __restrict__ cnt, long long cap,
                                                      double* __restrict__ partials) {
    __shared__ double s[NMI_BT / 32];
    const double dn = (double)n;
    const long long t0 = (long long)blockIdx.x * blockDim.x + threadIdx.x, nt = (long long)gridDim.x * blockDim.x;
    double I = 0, hx = 0, hy = 0;
    for (long long i = t0; i < cap; i += nt) {
        const ull k = keys[i];
        if (k == NMI_EMPTY) continue;
        const double nab = (double)cnt[i];
        const double pa = (double)na[k >> 32], pb = (double)nb[k & 0xFFFFFFFFull];
        I += nab / dn * log(dn * nab / (pa * pb));
    }
    for (long long i = t0; i < n; i += nt) {
        const unsigned a = na[i], b = nb[i];
        if (a) hx -= (double)a / dn * log((double)a / dn);
        if (b) hy -= (double)b / dn * log((double)b / dn);
    }
    I = nmi_block_sum(I, s);
    hx = nmi_block_sum(hx, s);
    hy = nmi_block_sum(hy, s);
    if (threadIdx.x == 0) {
        partials[3 * blockIdx.x] = I;
        partials[3 * blockIdx.x + 1] = hx;
        partials[3 * blockIdx.x + 2] = hy;
    }
}

// one thread: the block partials in block order, then the ratio and the degenerate convention
__global__ void k_nmi_final(const double* __restrict__ partials, int nblocks, double* __restrict__ out) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    double I = 0, hx = 0, hy = 0;
    for (int b = 0; b < nblocks; ++b) {
        I += partials[3 * b];
        hx += partials[3 * b + 1];
        hy += partials[3 * b + 2];
    }
    // a single cluster has H = 0 exactly: -(n/n) ln(n/n) = -1 * 0
    if (hx == 0.0 || hy == 0.0) *out = (hx == hy) ? 1.0 : 0.0;
    else *out = I / sqrt(hx * hy);
}
