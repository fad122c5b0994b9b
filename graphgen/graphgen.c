/*
 * graphgen.c — seeded synthetic graph generators and the CSR builder.
 *
 * This module is INPUT PLUMBING shared by the CPU oracle (oracle/) and the
 * CUDA path (paper_conf_ppopp_wangllwm00z25_b200/): it holds none of the
 * method's arithmetic (no modularity, no gains, no community logic).  Every
 * random draw is a pure function of (seed, stream, index) through a
 * counter-based generator (splitmix64 finaliser), so output is identical for
 * any OpenMP thread count.
 *
 * Generators (recipes: SURVEY.md §8(d)):
 *   - R-MAT (Chakrabarti et al.), quadrant probabilities (a,b,c,d), used for
 *     the LiveJournal-shaped config.
 *   - LFR-style planted partition (Lancichinetti-Fortunato-Radicchi [31],
 *     PAPER.md line 378 / Table 4), used for the LFR-1M, Orkut- and
 *     Friendster-shaped configs.
 *   - CSR builder: symmetrise, drop self loops, merge duplicates, sort rows.
 * The paper converts directed graphs to undirected before use (PAPER.md line
 * 340, §5); the builder does the same.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <omp.h>

/* ------------------------------------------------------------------------ */
/* counter-based RNG                                                         */
/* ------------------------------------------------------------------------ */
static inline uint64_t mix64(uint64_t z) {
    z += 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}
static inline uint64_t rng_u64(uint64_t seed, uint64_t stream, uint64_t idx) {
    return mix64(mix64(seed * 0x2545f4914f6cdd1dULL + stream) ^ (idx * 0x9e3779b97f4a7c15ULL + 0x632be59bd9b4e019ULL));
}
static inline double rng_unit(uint64_t seed, uint64_t stream, uint64_t idx) {
    return (double)(rng_u64(seed, stream, idx) >> 11) * (1.0 / 9007199254740992.0);
}

uint64_t gg_rng_u64(uint64_t seed, uint64_t stream, uint64_t idx) { return rng_u64(seed, stream, idx); }

/* ------------------------------------------------------------------------ */
/* parallel stable LSD radix sort of (key, val) uint64 pairs                 */
/* ------------------------------------------------------------------------ */
static void radix_sort_pairs(uint64_t* key, uint64_t* val, int64_t n, int key_bits) {
    if (n <= 1) return;
    uint64_t* k2 = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
    uint64_t* v2 = val ? (uint64_t*)malloc((size_t)n * sizeof(uint64_t)) : NULL;
    int nt = omp_get_max_threads();
    if (n < 1 << 16) nt = 1;
    int64_t* hist = (int64_t*)malloc((size_t)nt * 256 * sizeof(int64_t));
    uint64_t *ks = key, *vs = val, *kd = k2, *vd = v2;
    int passes = (key_bits + 7) / 8;
    for (int p = 0; p < passes; ++p) {
        int sh = p * 8;
        memset(hist, 0, (size_t)nt * 256 * sizeof(int64_t));
        #pragma omp parallel num_threads(nt)
        {
            int t = omp_get_thread_num();
            int64_t lo = n * t / nt, hi = n * (t + 1) / nt;
            int64_t* h = hist + (size_t)t * 256;
            for (int64_t i = lo; i < hi; ++i) h[(ks[i] >> sh) & 255]++;
            #pragma omp barrier
            #pragma omp single
            {
                int64_t run = 0;
                for (int b = 0; b < 256; ++b)
                    for (int tt = 0; tt < nt; ++tt) {
                        int64_t c = hist[(size_t)tt * 256 + b];
                        hist[(size_t)tt * 256 + b] = run;
                        run += c;
                    }
            }
            for (int64_t i = lo; i < hi; ++i) {
                int64_t dst = h[(ks[i] >> sh) & 255]++;
                kd[dst] = ks[i];
                if (vs) vd[dst] = vs[i];
            }
        }
        uint64_t* t = ks; ks = kd; kd = t;
        t = vs; vs = vd; vd = t;
    }
    if (ks != key) {
        memcpy(key, ks, (size_t)n * sizeof(uint64_t));
        if (val) memcpy(val, vs, (size_t)n * sizeof(uint64_t));
    }
    free(hist);
    free(k2);
    free(v2);
}

static int bits_for(uint64_t x) { int b = 1; while (b < 64 && (x >> b)) ++b; return b; }

/* ------------------------------------------------------------------------ */
/* CSR builder                                                               */
/* ------------------------------------------------------------------------ */
/*
 * gg_build_csr: undirected edge list (src[i], dst[i], w[i] or 1) -> symmetric
 * CSR with rows sorted by column.  Each input pair (u,v), u != v, yields the
 * two entries (u,v) and (v,u).  A self loop (v,v,w) yields ONE entry (v,v,w)
 * when keep_self_loops != 0, else it is dropped.  Duplicate entries are merged
 * (weights summed) when merge_dups != 0, else kept.
 * Output arrays must hold 2*m entries; row_ptr holds n+1.  Returns nnz, or -1
 * on an out-of-range endpoint.
 */
int64_t gg_build_csr(int64_t n, int64_t m, const int64_t* src, const int64_t* dst,
                     const int64_t* w, int keep_self_loops, int merge_dups,
                     int64_t* row_ptr, int32_t* col, int64_t* wout) {
    int kb = bits_for((uint64_t)(n > 1 ? n - 1 : 1));
    uint64_t* key = (uint64_t*)malloc((size_t)(2 * m + 1) * sizeof(uint64_t));
    uint64_t* val = (uint64_t*)malloc((size_t)(2 * m + 1) * sizeof(uint64_t));
    int64_t bad = 0;
    /* count entries per input edge to get write offsets deterministically */
    int64_t* cnt = (int64_t*)malloc((size_t)(m + 1) * sizeof(int64_t));
    #pragma omp parallel for reduction(+:bad)
    for (int64_t i = 0; i < m; ++i) {
        int64_t u = src[i], v = dst[i];
        if (u < 0 || u >= n || v < 0 || v >= n) { bad++; cnt[i] = 0; continue; }
        cnt[i] = (u == v) ? (keep_self_loops ? 1 : 0) : 2;
    }
    if (bad) { free(key); free(val); free(cnt); return -1; }
    int64_t tot = 0;
    for (int64_t i = 0; i < m; ++i) { int64_t c = cnt[i]; cnt[i] = tot; tot += c; }
    #pragma omp parallel for
    for (int64_t i = 0; i < m; ++i) {
        uint64_t u = (uint64_t)src[i], v = (uint64_t)dst[i];
        uint64_t ww = w ? (uint64_t)w[i] : 1;
        int64_t o = cnt[i];
        if (u == v) {
            if (keep_self_loops) { key[o] = (u << kb) | v; val[o] = ww; }
        } else {
            key[o] = (u << kb) | v; val[o] = ww;
            key[o + 1] = (v << kb) | u; val[o + 1] = ww;
        }
    }
    free(cnt);
    radix_sort_pairs(key, val, tot, 2 * kb);
    /* merge duplicates (sequential compaction; keys sorted) */
    int64_t nnz = 0;
    for (int64_t i = 0; i < tot; ++i) {
        if (merge_dups && nnz > 0 && key[nnz - 1] == key[i]) { val[nnz - 1] += val[i]; continue; }
        key[nnz] = key[i]; val[nnz] = val[i]; ++nnz;
    }
    uint64_t mask = (kb >= 64) ? ~0ULL : ((1ULL << kb) - 1);
    for (int64_t v = 0; v <= n; ++v) row_ptr[v] = 0;
    for (int64_t i = 0; i < nnz; ++i) row_ptr[(key[i] >> kb) + 1]++;
    for (int64_t v = 0; v < n; ++v) row_ptr[v + 1] += row_ptr[v];
    #pragma omp parallel for
    for (int64_t i = 0; i < nnz; ++i) {
        col[i] = (int32_t)(key[i] & mask);
        if (wout) wout[i] = (int64_t)val[i];
    }
    free(key);
    free(val);
    return nnz;
}

/* ------------------------------------------------------------------------ */
/* random permutation (sort of indices by a keyed hash)                      */
/* ------------------------------------------------------------------------ */
void gg_random_permutation(int64_t n, uint64_t seed, uint64_t stream, int64_t* perm) {
    uint64_t* k = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
    uint64_t* v = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
    #pragma omp parallel for
    for (int64_t i = 0; i < n; ++i) { k[i] = rng_u64(seed, stream, (uint64_t)i); v[i] = (uint64_t)i; }
    radix_sort_pairs(k, v, n, 64);
    #pragma omp parallel for
    for (int64_t i = 0; i < n; ++i) perm[v[i]] = i;   /* vertex v[i] gets new id i */
    free(k);
    free(v);
}

/* ------------------------------------------------------------------------ */
/* R-MAT                                                                     */
/* ------------------------------------------------------------------------ */
/*
 * gg_rmat: candidate edge e (0,1,2,...) descends `scale` levels choosing a
 * quadrant with probabilities (a, b, c, 1-a-b-c) using draw (seed, 10+level, e).
 * Endpoints >= n and self pairs are rejected.  Undirected duplicates are
 * removed and the first `target` distinct edges in candidate-index order are
 * kept.  Endpoints are then relabelled by a seeded random permutation so id
 * locality does not flatter the gathers.  Output: out_src/out_dst (target
 * entries each).  Returns the number of edges produced (<= target).
 */
int64_t gg_rmat(int scale, int64_t n, double a, double b, double c, uint64_t seed,
                int64_t target, int64_t* out_src, int64_t* out_dst) {
    int kb = bits_for((uint64_t)(n - 1));
    int64_t have = 0;
    int64_t next_idx = 0;
    /* accumulated distinct edges: key=(min<<kb|max), val=first idx */
    uint64_t* ak = NULL; uint64_t* av = NULL; int64_t acap = 0;
    double ab = a + b, abc = a + b + c;
    while (have < target) {
        int64_t batch = (int64_t)((double)(target - have) * 1.25) + 1024;
        int64_t tot = have + batch;
        if (tot > acap) {
            acap = tot;
            ak = (uint64_t*)realloc(ak, (size_t)acap * sizeof(uint64_t));
            av = (uint64_t*)realloc(av, (size_t)acap * sizeof(uint64_t));
        }
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < batch; ++i) {
            uint64_t e = (uint64_t)(next_idx + i);
            uint64_t u = 0, v = 0;
            for (int l = 0; l < scale; ++l) {
                double r = rng_unit(seed, 10 + (uint64_t)l, e);
                u <<= 1; v <<= 1;
                if (r < a) { }
                else if (r < ab) { v |= 1; }
                else if (r < abc) { u |= 1; }
                else { u |= 1; v |= 1; }
            }
            uint64_t k;
            if (u == v || u >= (uint64_t)n || v >= (uint64_t)n) k = ~0ULL;
            else k = (u < v) ? ((u << kb) | v) : ((v << kb) | u);
            ak[have + i] = k;
            av[have + i] = e;
        }
        next_idx += batch;
        /* sort by idx is the arrival order already; stable radix sort by key keeps idx order */
        radix_sort_pairs(ak, av, tot, 64);
        int64_t w = 0;
        for (int64_t i = 0; i < tot; ++i) {
            if (ak[i] == ~0ULL) break;
            if (w > 0 && ak[w - 1] == ak[i]) {
                if (av[i] < av[w - 1]) av[w - 1] = av[i];
                continue;
            }
            ak[w] = ak[i]; av[w] = av[i]; ++w;
        }
        have = w;
    }
    /* keep first `target` by idx: sort by idx */
    radix_sort_pairs(av, ak, have, 64);
    int64_t out = have < target ? have : target;
    int64_t* perm = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    gg_random_permutation(n, seed, 99, perm);
    uint64_t mask = (1ULL << kb) - 1;
    #pragma omp parallel for
    for (int64_t i = 0; i < out; ++i) {
        out_src[i] = perm[ak[i] >> kb];
        out_dst[i] = perm[ak[i] & mask];
    }
    free(perm);
    free(ak);
    free(av);
    return out;
}

/* ------------------------------------------------------------------------ */
/* LFR-style planted partition                                               */
/* ------------------------------------------------------------------------ */
static double pl_mean(int64_t kmin, int64_t kmax, double tau) {
    double s = 0, sk = 0;
    for (int64_t k = kmin; k <= kmax; ++k) { double p = pow((double)k, -tau); s += p; sk += p * (double)k; }
    return sk / s;
}
/* cumulative table of a discrete power law on [lo, hi] */
static double* pl_table(int64_t lo, int64_t hi, double tau) {
    int64_t m = hi - lo + 1;
    double* t = (double*)malloc((size_t)m * sizeof(double));
    double s = 0;
    for (int64_t i = 0; i < m; ++i) { s += pow((double)(lo + i), -tau); t[i] = s; }
    for (int64_t i = 0; i < m; ++i) t[i] /= s;
    return t;
}
static int64_t pl_draw(const double* t, int64_t lo, int64_t hi, double u) {
    int64_t l = 0, h = hi - lo;
    while (l < h) { int64_t mid = (l + h) / 2; if (t[mid] < u) l = mid + 1; else h = mid; }
    return lo + l;
}

/* ------------------------------------------------------------------------ */
/* degree-preserving rewiring of a configuration-model edge list             */
/* ------------------------------------------------------------------------ */
/* open-addressing set of undirected edge keys (min << 32 | max) with tombstones */
#define ES_EMPTY (~0ULL)
#define ES_TOMB (~1ULL)
typedef struct { uint64_t* t; uint64_t mask; } edgeset;
static inline uint64_t ekey(int64_t u, int64_t v) {
    return u < v ? ((uint64_t)u << 32) | (uint64_t)v : ((uint64_t)v << 32) | (uint64_t)u;
}
static inline uint64_t es_slot(uint64_t k) { return mix64(k); }
static int es_has(const edgeset* s, uint64_t k) {
    for (uint64_t i = es_slot(k) & s->mask;; i = (i + 1) & s->mask) {
        if (s->t[i] == k) return 1;
        if (s->t[i] == ES_EMPTY) return 0;
    }
}
static int es_insert(edgeset* s, uint64_t k) {   /* 0 if already present */
    uint64_t tomb = ES_EMPTY;
    for (uint64_t i = es_slot(k) & s->mask;; i = (i + 1) & s->mask) {
        if (s->t[i] == k) return 0;
        if (s->t[i] == ES_TOMB && tomb == ES_EMPTY) tomb = i;
        if (s->t[i] == ES_EMPTY) { s->t[tomb != ES_EMPTY ? tomb : i] = k; return 1; }
    }
}
static void es_erase(edgeset* s, uint64_t k) {
    for (uint64_t i = es_slot(k) & s->mask;; i = (i + 1) & s->mask) {
        if (s->t[i] == k) { s->t[i] = ES_TOMB; return; }
        if (s->t[i] == ES_EMPTY) return;
    }
}

/*
 * Edges [0, n_int) are internal, grouped by community (community j owns
 * [ioff[j], ioff[j+1])); edges [n_int, ne) are external.  An edge is bad if it
 * is a self pair, repeats an earlier edge, or (external) joins one community.
 * Each bad edge (u, v), in index order, is swapped with a random good edge
 * (c, d) of its class -> (u, d), (c, v) when both are new, distinct, non-self
 * and (external) cross communities; every vertex keeps its internal and
 * external degree.  Up to 256 draws per bad edge (stream 20), then it is
 * dropped.  Sequential, so the output is a pure function of the seed.
 * Returns the compacted edge count.
 */
static int64_t lfr_rewire(int64_t ne, int64_t n_int, int64_t* src, int64_t* dst, const int64_t* comm,
                          const int64_t* ioff, uint64_t seed) {
    uint64_t cap = 1024;
    while (cap < (uint64_t)(2 * ne + 2)) cap <<= 1;
    edgeset s = { (uint64_t*)malloc(cap * sizeof(uint64_t)), cap - 1 };
    memset(s.t, 0xff, cap * sizeof(uint64_t));
    unsigned char* bad = (unsigned char*)calloc((size_t)ne + 1, 1);
    for (int64_t e = 0; e < ne; ++e) {
        const int64_t u = src[e], v = dst[e];
        if (u == v || (e >= n_int && comm[u] == comm[v]) || !es_insert(&s, ekey(u, v))) bad[e] = 1;
    }
    const int64_t n_ext = ne - n_int;
    for (int64_t e = 0; e < ne; ++e) {
        if (!bad[e]) continue;
        const int64_t u = src[e], v = dst[e];
        const int internal = e < n_int;
        int64_t lo, len;
        if (internal) { const int64_t c = comm[u]; lo = ioff[c]; len = ioff[c + 1] - lo; }
        else { lo = n_int; len = n_ext; }
        if (len < 2) continue;
        for (uint64_t t = 0; t < 256; ++t) {
            const uint64_t r = rng_u64(seed, 20, ((uint64_t)e << 8) | t);
            const int64_t j = lo + (int64_t)((r >> 1) % (uint64_t)len);
            if (j == e || bad[j]) continue;
            int64_t c = src[j], d = dst[j];
            if (r & 1) { const int64_t x = c; c = d; d = x; }
            if (u == d || c == v) continue;
            if (!internal && (comm[u] == comm[d] || comm[c] == comm[v])) continue;
            const uint64_t k1 = ekey(u, d), k2 = ekey(c, v);
            if (k1 == k2 || es_has(&s, k1) || es_has(&s, k2)) continue;
            es_erase(&s, ekey(c, d));
            es_insert(&s, k1);
            es_insert(&s, k2);
            src[e] = u; dst[e] = d;
            src[j] = c; dst[j] = v;
            bad[e] = 0;
            break;
        }
    }
    int64_t w = 0;
    for (int64_t e = 0; e < ne; ++e)
        if (!bad[e]) { src[w] = src[e]; dst[w] = dst[e]; ++w; }
    free(bad);
    free(s.t);
    return w;
}

/*
 * gg_lfr: LFR-style benchmark graph.
 *   1. degrees k_i ~ discrete power law (tau1) on [kmin, kmax]; kmin is the
 *      integer whose mean is closest to avg_k (stream 1).
 *   2. community sizes ~ discrete power law (tau2) on [cmin, cmax] until they
 *      cover n (stream 2); the remainder is spread one vertex at a time.
 *   3. k_in = round((1-mu) k), k_out = k - k_in.
 *   4. vertices in decreasing k_in (ties by id) are placed in random
 *      communities with spare capacity and size > k_in (stream 3).
 *   5. internal stubs are paired by a seeded shuffle per community (stream 4);
 *      external stubs by a global seeded shuffle (stream 5), re-pairing the
 *      pairs that fell inside one community twice (streams 6,7), then dropping.
 *   6. ids are permuted (stream 8).
 * Output: edges (u, v) (possibly with self pairs/duplicates — the CSR builder
 * removes them), membership[n] (ground truth, permuted ids).
 * Two-call protocol: if out_src == NULL returns the edge count upper bound.
 */
/* LFR plan (steps 1-4 of gg_lfr_ex): degrees k, and unless degrees_only, community sizes, internal
   degrees kin, the placement comm and the per-community member lists (coff, mem).  Shared by
   gg_lfr_ex and the memory-lean gg_lfr_csr. */
typedef struct {
    int64_t kmin, stubs_total, nc, maxc;
    int64_t *k, *kin, *csize, *fill, *comm, *coff, *mem;
} lfr_plan_t;

static void lfr_plan_free(lfr_plan_t* P) {
    free(P->k); free(P->kin); free(P->csize); free(P->fill); free(P->comm); free(P->coff); free(P->mem);
}

static void lfr_plan(int64_t n, double avg_k, int64_t kmax, double tau1, double tau2, int64_t cmin, int64_t cmax,
                     double mu, uint64_t seed, int fit_frac, double alpha, int degrees_only, lfr_plan_t* P) {
    memset(P, 0, sizeof(*P));
    /* 1. degrees */
    int64_t best_kmin = 1; double best_err = 1e300;
    for (int64_t km = 1; km < kmax; ++km) {
        double e = fabs(pl_mean(km, kmax, tau1) - avg_k);
        if (e < best_err) { best_err = e; best_kmin = km; }
    }
    int64_t kmin = best_kmin;
    double* tk;
    if (fit_frac) {
        /* exact mean: the law on [K0, kmax] with the weight of k = K0 scaled by f in (0, 1],
           K0 the largest integer whose full law has mean <= avg_k; f by bisection */
        int64_t k0 = 1;
        while (k0 + 1 < kmax && pl_mean(k0 + 1, kmax, tau1) <= avg_k) ++k0;
        double lo = 1e-9, hi = 1.0, f = 1.0;
        double s_rest = 0, sk_rest = 0;
        for (int64_t k = k0 + 1; k <= kmax; ++k) { double p = pow((double)k, -tau1); s_rest += p; sk_rest += p * (double)k; }
        const double p0 = pow((double)k0, -tau1);
        for (int it = 0; it < 200; ++it) {
            f = 0.5 * (lo + hi);
            const double m = (sk_rest + f * p0 * (double)k0) / (s_rest + f * p0);
            if (m > avg_k) lo = f; else hi = f;   /* larger f -> more mass at k0 -> smaller mean */
        }
        kmin = k0;
        tk = pl_table(kmin, kmax, tau1);
        const int64_t m = kmax - kmin + 1;
        double s = s_rest + f * p0, acc = f * p0;
        tk[0] = acc / s;
        for (int64_t i = 1; i < m; ++i) { acc += pow((double)(kmin + i), -tau1); tk[i] = acc / s; }
        tk[m - 1] = 1.0;
    } else {
        tk = pl_table(kmin, kmax, tau1);
    }
    P->kmin = kmin;
    int64_t* k = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    #pragma omp parallel for
    for (int64_t i = 0; i < n; ++i) k[i] = pl_draw(tk, kmin, kmax, rng_unit(seed, 1, (uint64_t)i));
    free(tk);
    int64_t stubs_total = 0;
    for (int64_t i = 0; i < n; ++i) stubs_total += k[i];
    P->k = k;
    P->stubs_total = stubs_total;
    if (degrees_only) return;

    /* 2. community sizes */
    double* tc = pl_table(cmin, cmax, tau2);
    int64_t ccap = n / cmin + 2;
    int64_t* csize = (int64_t*)malloc((size_t)ccap * sizeof(int64_t));
    int64_t nc = 0, covered = 0;
    while (covered < n) {
        int64_t s = pl_draw(tc, cmin, cmax, rng_unit(seed, 2, (uint64_t)nc));
        if (covered + s > n) s = n - covered;
        csize[nc++] = s; covered += s;
    }
    free(tc);
    if (nc > 1 && csize[nc - 1] < cmin) {   /* spread a short remainder */
        int64_t r = csize[--nc];
        for (int64_t j = 0; r > 0; j = (j + 1) % nc) { if (csize[j] < cmax) { csize[j]++; r--; } }
    }
    int64_t maxc = 0;
    for (int64_t j = 0; j < nc; ++j) if (csize[j] > maxc) maxc = csize[j];

    /* 3. internal / external degrees */
    int64_t* kin = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    for (int64_t i = 0; i < n; ++i) {
        int64_t ki = (int64_t)llround((1.0 - mu) * (double)k[i]);
        const int64_t cap = (int64_t)floor(alpha * (double)(maxc - 1));
        if (ki > cap) ki = cap;   /* the excess becomes external stubs (k_out = k - k_in) */
        kin[i] = ki;
    }

    /* 4. placement: order by k_in desc (radix sort on (kmax - kin, id)) */
    uint64_t* ok = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
    uint64_t* ov = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
    for (int64_t i = 0; i < n; ++i) { ok[i] = (uint64_t)(maxc - kin[i]); ov[i] = (uint64_t)i; }
    radix_sort_pairs(ok, ov, n, bits_for((uint64_t)maxc));
    int64_t* fill = (int64_t*)calloc((size_t)nc, sizeof(int64_t));
    int64_t* comm = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    for (int64_t t = 0; t < n; ++t) {
        int64_t v = (int64_t)ov[t];
        int64_t chosen = -1;
        for (int tr = 0; tr < 64 && chosen < 0; ++tr) {
            int64_t c = (int64_t)(rng_u64(seed, 3, (uint64_t)t * 64 + (uint64_t)tr) % (uint64_t)nc);
            if (fill[c] < csize[c] && alpha * (double)(csize[c] - 1) >= (double)kin[v]) chosen = c;
        }
        if (chosen < 0) {   /* deterministic scan fallback */
            int64_t st = (int64_t)(rng_u64(seed, 3, (uint64_t)t * 64 + 63) % (uint64_t)nc);
            for (int64_t j = 0; j < nc && chosen < 0; ++j) {
                int64_t c = (st + j) % nc;
                if (fill[c] < csize[c] && alpha * (double)(csize[c] - 1) >= (double)kin[v]) chosen = c;
            }
            if (chosen < 0) {   /* no community large enough: any with room; cap k_in */
                for (int64_t j = 0; j < nc && chosen < 0; ++j) {
                    int64_t c = (st + j) % nc;
                    if (fill[c] < csize[c]) chosen = c;
                }
                {
                    const int64_t cap = (int64_t)floor(alpha * (double)(csize[chosen] - 1));
                    if (kin[v] > cap) kin[v] = cap;   /* excess -> external stubs */
                }
            }
        }
        comm[v] = chosen;
        fill[chosen]++;
    }
    free(ok); free(ov);

    /* members list per community (by id order) */
    int64_t* coff = (int64_t*)calloc((size_t)nc + 1, sizeof(int64_t));
    for (int64_t i = 0; i < n; ++i) coff[comm[i] + 1]++;
    for (int64_t j = 0; j < nc; ++j) coff[j + 1] += coff[j];
    int64_t* mem = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    {
        int64_t* cur = (int64_t*)malloc((size_t)nc * sizeof(int64_t));
        memcpy(cur, coff, (size_t)nc * sizeof(int64_t));
        for (int64_t i = 0; i < n; ++i) mem[cur[comm[i]]++] = i;
        free(cur);
    }
    P->kin = kin; P->csize = csize; P->fill = fill; P->comm = comm; P->coff = coff; P->mem = mem;
    P->nc = nc; P->maxc = maxc;
}

int64_t gg_lfr_ex(int64_t n, double avg_k, int64_t kmax, double tau1, double tau2,
                  int64_t cmin, int64_t cmax, double mu, uint64_t seed, int fit_frac, double alpha,
                  int rewire, int64_t* out_src, int64_t* out_dst, int64_t* membership, int64_t* out_kmin) {
    lfr_plan_t P;
    lfr_plan(n, avg_k, kmax, tau1, tau2, cmin, cmax, mu, seed, fit_frac, alpha, out_src == NULL, &P);
    if (out_kmin) *out_kmin = P.kmin;
    if (!out_src) { lfr_plan_free(&P); return P.stubs_total / 2 + n; }
    int64_t *k = P.k, *kin = P.kin, *comm = P.comm, *coff = P.coff, *mem = P.mem;
    const int64_t nc = P.nc;

    /* 5a. internal wiring: per community stub shuffle */
    int64_t* istub_off = (int64_t*)calloc((size_t)nc + 1, sizeof(int64_t));
    for (int64_t j = 0; j < nc; ++j) {
        int64_t s = 0;
        for (int64_t t = coff[j]; t < coff[j + 1]; ++t) s += kin[mem[t]];
        istub_off[j + 1] = istub_off[j] + s / 2;   /* number of internal edges */
    }
    int64_t n_int = istub_off[nc];
    int64_t n_out_stubs = 0;
    for (int64_t i = 0; i < n; ++i) n_out_stubs += k[i] - kin[i];
    int64_t ne = 0;
    #pragma omp parallel
    {
        int64_t bufcap = 0; int64_t* buf = NULL;
        #pragma omp for schedule(dynamic, 16)
        for (int64_t j = 0; j < nc; ++j) {
            int64_t s = 0;
            for (int64_t t = coff[j]; t < coff[j + 1]; ++t) s += kin[mem[t]];
            if (s > bufcap) { bufcap = s; buf = (int64_t*)realloc(buf, (size_t)bufcap * sizeof(int64_t)); }
            int64_t p = 0;
            for (int64_t t = coff[j]; t < coff[j + 1]; ++t)
                for (int64_t q = 0; q < kin[mem[t]]; ++q) buf[p++] = mem[t];
            for (int64_t i = s - 1; i > 0; --i) {   /* Fisher-Yates, keyed draws */
                int64_t r = (int64_t)(rng_u64(seed, 4, ((uint64_t)j << 32) ^ (uint64_t)i) % (uint64_t)(i + 1));
                int64_t tmp = buf[i]; buf[i] = buf[r]; buf[r] = tmp;
            }
            int64_t o = istub_off[j];
            for (int64_t e = 0; e < s / 2; ++e) { out_src[o + e] = buf[2 * e]; out_dst[o + e] = buf[2 * e + 1]; }
        }
        free(buf);
    }
    ne = n_int;

    /* 5b. external wiring: global shuffle via sort by keyed hash */
    uint64_t* sk = (uint64_t*)malloc((size_t)(n_out_stubs + 1) * sizeof(uint64_t));
    uint64_t* sv = (uint64_t*)malloc((size_t)(n_out_stubs + 1) * sizeof(uint64_t));
    {
        int64_t p = 0;
        for (int64_t i = 0; i < n; ++i)
            for (int64_t q = 0; q < k[i] - kin[i]; ++q) { sv[p] = (uint64_t)i; ++p; }
        #pragma omp parallel for
        for (int64_t i = 0; i < n_out_stubs; ++i) sk[i] = rng_u64(seed, 5, (uint64_t)i);
        radix_sort_pairs(sk, sv, n_out_stubs, 64);
    }
    int64_t np = n_out_stubs / 2;
    for (int round = 0; round < 2; ++round) {
        /* collect stubs of bad pairs, reshuffle them among themselves */
        int64_t nb = 0;
        for (int64_t e = 0; e < np; ++e)
            if (comm[sv[2 * e]] == comm[sv[2 * e + 1]]) nb++;
        if (nb == 0) break;
        uint64_t* bk = (uint64_t*)malloc((size_t)(2 * nb) * sizeof(uint64_t));
        uint64_t* bv = (uint64_t*)malloc((size_t)(2 * nb) * sizeof(uint64_t));
        int64_t* pos = (int64_t*)malloc((size_t)(2 * nb) * sizeof(int64_t));
        int64_t b = 0;
        for (int64_t e = 0; e < np; ++e)
            if (comm[sv[2 * e]] == comm[sv[2 * e + 1]]) {
                pos[b] = 2 * e; bv[b] = sv[2 * e]; bk[b] = rng_u64(seed, 6 + (uint64_t)round, (uint64_t)b); ++b;
                pos[b] = 2 * e + 1; bv[b] = sv[2 * e + 1]; bk[b] = rng_u64(seed, 6 + (uint64_t)round, (uint64_t)b); ++b;
            }
        radix_sort_pairs(bk, bv, b, 64);
        for (int64_t i = 0; i < b; ++i) sv[pos[i]] = bv[i];
        free(bk); free(bv); free(pos);
    }
    for (int64_t e = 0; e < np; ++e) {
        int64_t u = (int64_t)sv[2 * e], v = (int64_t)sv[2 * e + 1];
        if (comm[u] == comm[v] && !rewire) continue;   /* dropped after two re-pairings */
        out_src[ne] = u; out_dst[ne] = v; ++ne;
    }
    free(sk); free(sv);
    /* 5c. (rewire) degree-preserving double-edge swaps replace self pairs, duplicates and
       external pairs inside one community instead of dropping them */
    if (rewire) ne = lfr_rewire(ne, n_int, out_src, out_dst, comm, istub_off, seed);

    /* 6. permute ids */
    int64_t* perm = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    gg_random_permutation(n, seed, 8, perm);
    #pragma omp parallel for
    for (int64_t e = 0; e < ne; ++e) { out_src[e] = perm[out_src[e]]; out_dst[e] = perm[out_dst[e]]; }
    if (membership) {
        #pragma omp parallel for
        for (int64_t i = 0; i < n; ++i) membership[perm[i]] = comm[i];
    }
    free(perm); lfr_plan_free(&P); free(istub_off);
    return ne;
}

/* the original entry point: integer k_min, internal degree capped at community size - 1 */
int64_t gg_lfr(int64_t n, double avg_k, int64_t kmax, double tau1, double tau2,
               int64_t cmin, int64_t cmax, double mu, uint64_t seed,
               int64_t* out_src, int64_t* out_dst, int64_t* membership, int64_t* out_kmin) {
    return gg_lfr_ex(n, avg_k, kmax, tau1, tau2, cmin, cmax, mu, seed, 0, 1.0, 0, out_src, out_dst, membership, out_kmin);
}

/* ---------------------------------------------------------------------------------------------
 * Memory-lean LFR-style generator straight to CSR, for graphs whose edge list does not fit the
 * host twice over (the Friendster shape: 65.6M vertices, ~1.8B edges).
 * Same plan as gg_lfr_ex (degrees, community sizes, placement, per-community internal wiring),
 * but the external stubs are paired through a counter-based random bijection of the stub
 * sequence instead of a sort by random key: stub j of the shuffled sequence is pi(j), pi a
 * 4-round Feistel permutation of [0, 2^2h) restricted to [0, S) by cycle walking, and pair e is
 * (pi(2e), pi(2e+1)).  Every pair is a pure function of (seed, e), so the O(S) stub arrays and
 * their sort buffers are never built.  External pairs inside one community, self pairs and
 * duplicate edges are dropped (no re-pairing, no rewiring; realised counts reported).
 * Peak host memory ~ 8 B per edge (packed edge list) + 4 B per CSR entry + O(n).
 * Returns nnz; *out_col receives a malloc'd int32[nnz] (free with gg_free), row_ptr is int64[n+1].
 * -------------------------------------------------------------------------------------------*/
static inline uint64_t feistel_perm(uint64_t x, uint64_t S, int half, uint64_t seed) {
    const uint64_t mask = (1ull << half) - 1;
    do {
        uint64_t L = x >> half, R = x & mask;
        for (int r = 0; r < 4; ++r) {
            const uint64_t F = mix64(R ^ (seed * 0x9E3779B97F4A7C15ull) ^ ((uint64_t)(r + 1) << 56)) & mask;
            const uint64_t t = L ^ F;
            L = R;
            R = t;
        }
        x = (L << half) | R;
    } while (x >= S);   /* cycle walking: a bijection of [0, S) */
    return x;
}

static int64_t stub_owner(const int64_t* off, int64_t n, uint64_t s) {   /* largest v with off[v] <= s */
    int64_t lo = 0, hi = n - 1;
    while (lo < hi) {
        const int64_t mid = (lo + hi + 1) / 2;
        if ((uint64_t)off[mid] <= s) lo = mid; else hi = mid - 1;
    }
    return lo;
}

static int cmp_i32(const void* a, const void* b) {
    const int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

void gg_free(void* p) { free(p); }

int64_t gg_lfr_csr(int64_t n, double avg_k, int64_t kmax, double tau1, double tau2, int64_t cmin, int64_t cmax,
                   double mu, uint64_t seed, int fit_frac, int64_t* row_ptr, int32_t** out_col, int64_t* membership,
                   int64_t* out_kmin, int64_t* out_stats /* [internal edges, external pairs, dropped] */) {
    lfr_plan_t P;
    lfr_plan(n, avg_k, kmax, tau1, tau2, cmin, cmax, mu, seed, fit_frac, 1.0, 0, &P);
    if (out_kmin) *out_kmin = P.kmin;
    int64_t *k = P.k, *kin = P.kin, *comm = P.comm, *coff = P.coff, *mem = P.mem;
    const int64_t nc = P.nc;
    /* internal edges per community */
    int64_t* ioff = (int64_t*)calloc((size_t)nc + 1, sizeof(int64_t));
    for (int64_t j = 0; j < nc; ++j) {
        int64_t s = 0;
        for (int64_t t = coff[j]; t < coff[j + 1]; ++t) s += kin[mem[t]];
        ioff[j + 1] = ioff[j] + s / 2;
    }
    const int64_t n_int = ioff[nc];
    int64_t* xoff = (int64_t*)malloc((size_t)(n + 1) * sizeof(int64_t));   /* external stub prefix */
    xoff[0] = 0;
    for (int64_t i = 0; i < n; ++i) xoff[i + 1] = xoff[i] + (k[i] - kin[i]);
    const uint64_t S = (uint64_t)xoff[n];
    const int64_t np = (int64_t)(S / 2);
    int half = 1;
    while (half < 32 && (1ull << (2 * half)) < S) ++half;
    int64_t* perm = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    gg_random_permutation(n, seed, 8, perm);
    uint64_t* E = (uint64_t*)malloc((size_t)(n_int + np + 1) * sizeof(uint64_t));   /* (u << 32 | v), ids permuted */
    const uint64_t DROP = ~0ull;
    /* 5a. internal wiring (per-community Fisher-Yates of its stubs, as gg_lfr_ex) */
    #pragma omp parallel
    {
        int64_t bufcap = 0; int64_t* buf = NULL;
        #pragma omp for schedule(dynamic, 16)
        for (int64_t j = 0; j < nc; ++j) {
            int64_t s = 0;
            for (int64_t t = coff[j]; t < coff[j + 1]; ++t) s += kin[mem[t]];
            if (s > bufcap) { bufcap = s; buf = (int64_t*)realloc(buf, (size_t)bufcap * sizeof(int64_t)); }
            int64_t p = 0;
            for (int64_t t = coff[j]; t < coff[j + 1]; ++t)
                for (int64_t q = 0; q < kin[mem[t]]; ++q) buf[p++] = mem[t];
            for (int64_t i = s - 1; i > 0; --i) {
                int64_t r = (int64_t)(rng_u64(seed, 4, ((uint64_t)j << 32) ^ (uint64_t)i) % (uint64_t)(i + 1));
                int64_t tmp = buf[i]; buf[i] = buf[r]; buf[r] = tmp;
            }
            for (int64_t e = 0; e < s / 2; ++e) {
                const int64_t u = buf[2 * e], v = buf[2 * e + 1];
                E[ioff[j] + e] = u == v ? DROP : ((uint64_t)perm[u] << 32) | (uint64_t)perm[v];
            }
        }
        free(buf);
    }
    /* 5b. external pairs through the Feistel bijection */
    int64_t dropped_x = 0;
    #pragma omp parallel for reduction(+ : dropped_x) schedule(static, 1 << 16)
    for (int64_t e = 0; e < np; ++e) {
        const uint64_t a = feistel_perm(2 * (uint64_t)e, S, half, seed ^ 0x5A5Aull);
        const uint64_t b = feistel_perm(2 * (uint64_t)e + 1, S, half, seed ^ 0x5A5Aull);
        const int64_t u = stub_owner(xoff, n, a), v = stub_owner(xoff, n, b);
        if (u == v || comm[u] == comm[v]) { E[n_int + e] = DROP; ++dropped_x; continue; }
        E[n_int + e] = ((uint64_t)perm[u] << 32) | (uint64_t)perm[v];
    }
    const int64_t m = n_int + np;
    if (membership) {
        #pragma omp parallel for
        for (int64_t i = 0; i < n; ++i) membership[perm[i]] = comm[i];
    }
    free(xoff); free(perm); free(ioff); lfr_plan_free(&P);
    /* 6. CSR: count, scatter both directions, sort + dedup every row, compact */
    for (int64_t v = 0; v <= n; ++v) row_ptr[v] = 0;
    #pragma omp parallel for
    for (int64_t e = 0; e < m; ++e) {
        if (E[e] == DROP) continue;
        __atomic_fetch_add(&row_ptr[(E[e] >> 32) + 1], 1, __ATOMIC_RELAXED);
        __atomic_fetch_add(&row_ptr[(E[e] & 0xFFFFFFFFull) + 1], 1, __ATOMIC_RELAXED);
    }
    for (int64_t v = 0; v < n; ++v) row_ptr[v + 1] += row_ptr[v];
    const int64_t tot = row_ptr[n];
    int32_t* col = (int32_t*)malloc((size_t)(tot + 1) * sizeof(int32_t));
    int64_t* cur = (int64_t*)malloc((size_t)n * sizeof(int64_t));
    memcpy(cur, row_ptr, (size_t)n * sizeof(int64_t));
    #pragma omp parallel for
    for (int64_t e = 0; e < m; ++e) {
        if (E[e] == DROP) continue;
        const int64_t u = (int64_t)(E[e] >> 32), v = (int64_t)(E[e] & 0xFFFFFFFFull);
        col[__atomic_fetch_add(&cur[u], 1, __ATOMIC_RELAXED)] = (int32_t)v;
        col[__atomic_fetch_add(&cur[v], 1, __ATOMIC_RELAXED)] = (int32_t)u;
    }
    free(E);
    /* per row: sort, unique (cur[v] = its distinct count) */
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < n; ++v) {
        int32_t* r = col + row_ptr[v];
        const int64_t len = row_ptr[v + 1] - row_ptr[v];
        qsort(r, (size_t)len, sizeof(int32_t), cmp_i32);
        int64_t w = 0;
        for (int64_t i = 0; i < len; ++i) if (i == 0 || r[i] != r[i - 1]) r[w++] = r[i];
        cur[v] = w;
    }
    int64_t nnz = 0;   /* compact left to right (new start <= old start: memmove is safe in order) */
    for (int64_t v = 0; v < n; ++v) {
        const int64_t b = row_ptr[v];
        if (nnz != b) memmove(col + nnz, col + b, (size_t)cur[v] * sizeof(int32_t));
        row_ptr[v] = nnz;
        nnz += cur[v];
    }
    row_ptr[n] = nnz;
    free(cur);
    *out_col = (int32_t*)realloc(col, (size_t)(nnz + 1) * sizeof(int32_t));
    if (out_stats) { out_stats[0] = n_int; out_stats[1] = np; out_stats[2] = m - nnz / 2; }
    return nnz;
}
