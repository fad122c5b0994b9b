/*
 * gala_oracle.c — plain, slow, obviously-correct CPU oracle of GALA's Louvain
 * (Wang et al., "Swift Unfolding of Communities: GPU-Accelerated Louvain
 * Algorithm", PPoPP'25).  P:N below = /root/reference/PAPER.md line N.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py (cpu_baseline leg / --impl reference) may load this library.  It
 * shares no code, header, table or helper with the CUDA path.
 *
 * What it computes:
 *   - modularity Q_gamma = sum_C [ D_C(C)/2|E| - gamma (D_V(C)/2|E|)^2 ]
 *     (Eq. 1; gamma: P:49, reading c11), kept as the exact integer
 *     numerator N = q*W*sum_C D_C(C) - p*sum_C D_V(C)^2 with W = 2|E| = D_V(V)
 *      and gamma = p/q;
 *   - phase 1 (Alg. 1) as BSP supersteps: every vertex
 *     decides from the start-of-iteration state; DecideAndMove takes the
 *     argmax of the modularity gain (Eq. 2) over NEIGHBOURING
 *     communities only, relative to staying ("remove v first",
 *     reading c1), ties to the lowest community id (c4), Grappolo singleton
 *     swap suppression (P:141 footnote 1, reading c5);
 *   - optional MG pruning (Eq. 6/7; reading c2: d_{C[v]}(v)
 *     excludes the self loop; c3: min over non-empty communities);
 *   - convergence Delta Q < theta (Alg. 1 lines 12-13, P:88-89, P:115,
 *     theta = 1e-6 P:340; readings c6, c7, c14);
 *   - phase 2: community -> super vertex, inter-community weights
 *     summed into super edges, internal weight D_C(C) into ONE self loop
 *     (reading c10), super vertices numbered in min-member order (c9);
 *   - the multi-level loop "until modularity convergence" (c8).
 * All arithmetic on weights, gains and N is exact integer (int64 / __int128).
 *
 * Parity pins (tests/test_oracle_*.py): karate literature values, closed
 * forms (ring of cliques, singletons, all-in-one), networkx modularity,
 * gain-vs-brute-force-Q identity, iteration-1 closed form, invariants,
 * brute-force optimum on <= 12 vertices, pruning on == off (Theorem 6).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <omp.h>

typedef __int128 i128;

/* ---------------------------------------------------------------- results */
typedef struct {
    int32_t level, iter;
    int64_t n_level, n_active, n_pruned, n_moved, n_fn, n_fp;
    i128 N;
    int32_t* labels; /* level-local community of every level vertex after the iteration */
    unsigned char* pruned; /* trace >= 3: 1 iff the pruning rule made the vertex inactive */
} orc_rec;

typedef struct {
    int64_t n, nnz, iters;
    i128 N_start, N_end;
} orc_level;

typedef struct {
    int64_t n0, W, p, q;
    int32_t* lab;          /* final canonical labels of level-0 vertices */
    int64_t k;             /* number of communities */
    i128 N;                /* final numerator (re-verified on G0) */
    orc_rec* rec; int64_t nrec, caprec;
    orc_level* lev; int64_t nlev, caplev;
    int status;            /* 0 ok, 1 invalid, 2 overflow, 3 internal check failed */
} orc_result;

static void push_rec(orc_result* r, orc_rec x) {
    if (r->nrec == r->caprec) {
        r->caprec = r->caprec ? 2 * r->caprec : 64;
        r->rec = (orc_rec*)realloc(r->rec, (size_t)r->caprec * sizeof(orc_rec));
    }
    r->rec[r->nrec++] = x;
}
static void push_lev(orc_result* r, orc_level x) {
    if (r->nlev == r->caplev) {
        r->caplev = r->caplev ? 2 * r->caplev : 16;
        r->lev = (orc_level*)realloc(r->lev, (size_t)r->caplev * sizeof(orc_level));
    }
    r->lev[r->nlev++] = x;
}

/* ----------------------------------------------------- gamma = p/q (c11) */
static int64_t gcd64(int64_t a, int64_t b) { while (b) { int64_t t = a % b; a = b; b = t; } return a; }
/* gamma is quantised to round(gamma * 2^16) / 2^16 and reduced. */
void oracle_gamma_pq(double gamma, int64_t* p, int64_t* q) {
    int64_t pp = (int64_t)(gamma * 65536.0 + 0.5), qq = 65536;
    int64_t g = gcd64(pp, qq);
    if (g == 0) g = 1;
    *p = pp / g; *q = qq / g;
}

/* -------------------------------------------------------- a graph level */
typedef struct {
    int64_t n;
    int64_t* rp;   /* n+1 */
    int32_t* col;  /* nnz */
    int64_t* w;    /* nnz, never NULL inside the oracle */
} ograph;

/* ------------------------------------------------- modularity (Eq. 1) */
/*
 * N(labels) = q*W*sum_C D_C(C) - p*sum_C D_V(C)^2 where
 *   D_C(C) = sum_{v in C} d_C(v): weight of entries (v,u) with both ends in C,
 *            each internal undirected edge counted twice, a stored
 *            self loop once;
 *   D_V(C) = sum_{v in C} d(v).
 * Labels may be any ids in [0, n).
 */
static i128 modularity_num(const ograph* g, const int32_t* lab, int64_t W, int64_t p, int64_t q) {
    int64_t n = g->n;
    int64_t* DV = (int64_t*)calloc((size_t)n, sizeof(int64_t));
    int64_t DC = 0;
    for (int64_t v = 0; v < n; ++v)
        for (int64_t e = g->rp[v]; e < g->rp[v + 1]; ++e) {
            DV[lab[v]] += g->w[e];
            if (lab[g->col[e]] == lab[v]) DC += g->w[e];
        }
    i128 S2 = 0;
    for (int64_t c = 0; c < n; ++c) S2 += (i128)DV[c] * DV[c];
    free(DV);
    return (i128)q * W * DC - (i128)p * S2;
}

/* --------------------------------------------- DecideAndMove (Alg. 1 l.14) */
typedef struct { int32_t c; int64_t w; } cw_pair;
static int cmp_pair(const void* a, const void* b) {
    int32_t x = ((const cw_pair*)a)->c, y = ((const cw_pair*)b)->c;
    return (x > y) - (x < y);
}

/*
 * Returns the community v would move to (== C[v] to stay).  buf has room for
 * deg(v) pairs.  d_own_out receives the aggregated weight to C[v] (= d'(v)).
 *   score(c) = q*W*d_c(v) - p*Sig[c]*d(v)                 (Eq. 2 x q*W*|E|)
 *   stay     = q*W*d'(v)  - p*(Sig[C[v]] - d(v))*d(v)     (reading c1)
 */
static int32_t decide(const ograph* g, int64_t v, const int32_t* C, const int64_t* Sig,
                      const int32_t* size, const int64_t* d, const int64_t* dp,
                      int64_t W, int64_t p, int64_t q, cw_pair* buf, int64_t* d_own_out) {
    int64_t k = 0;
    for (int64_t e = g->rp[v]; e < g->rp[v + 1]; ++e) {
        if (g->col[e] == v) continue;               /* self loop is not a neighbour */
        buf[k].c = C[g->col[e]]; buf[k].w = g->w[e]; ++k;
    }
    qsort(buf, (size_t)k, sizeof(cw_pair), cmp_pair);
    int32_t own = C[v];
    i128 stay = (i128)q * W * dp[v] - (i128)p * (Sig[own] - d[v]) * d[v];
    int32_t best = own;
    i128 best_score = stay;
    int64_t d_own = 0;
    for (int64_t i = 0; i < k;) {                  /* groups in ascending community id */
        int32_t c = buf[i].c;
        int64_t wc = 0;
        while (i < k && buf[i].c == c) { wc += buf[i].w; ++i; }
        if (c == own) { d_own = wc; continue; }
        i128 sc = (i128)q * W * wc - (i128)p * Sig[c] * d[v];
        if (sc > best_score) { best_score = sc; best = c; }   /* strict: ties keep lower id / stay */
    }
    /* Grappolo singleton swap suppression (reading c5) */
    if (best != own && size[best] == 1 && size[own] == 1 && best > own) best = own;
    *d_own_out = d_own;
    return best;
}

/* --------------------------------------------------- phase 2 */
/* coarse graph: vertex newid[v]; entry (newid[v], newid[u], w) summed by pair */
static void coarsen(const ograph* g, const int32_t* newid, int64_t k, ograph* out) {
    int64_t n = g->n;
    int64_t* cnt = (int64_t*)calloc((size_t)k + 1, sizeof(int64_t));
    for (int64_t v = 0; v < n; ++v) cnt[newid[v] + 1] += g->rp[v + 1] - g->rp[v];
    for (int64_t c = 0; c < k; ++c) cnt[c + 1] += cnt[c];
    int64_t tot = cnt[k];
    /* bucket the entries (coarse dst, w) by coarse source */
    cw_pair* ent = (cw_pair*)malloc((size_t)(tot + 1) * sizeof(cw_pair));
    int64_t* cur = (int64_t*)malloc((size_t)(k + 1) * sizeof(int64_t));
    memcpy(cur, cnt, (size_t)(k + 1) * sizeof(int64_t));
    for (int64_t v = 0; v < n; ++v)
        for (int64_t e = g->rp[v]; e < g->rp[v + 1]; ++e) {
            int64_t o = cur[newid[v]]++;
            ent[o].c = newid[g->col[e]];
            ent[o].w = g->w[e];
        }
    /* per coarse row: sort by destination, sum equal destinations in place */
    int64_t* rowlen = (int64_t*)calloc((size_t)k + 1, sizeof(int64_t));
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t c = 0; c < k; ++c) {
        int64_t lo = cnt[c], hi = cnt[c + 1];
        qsort(ent + lo, (size_t)(hi - lo), sizeof(cw_pair), cmp_pair);
        int64_t m = 0;
        for (int64_t i = lo; i < hi; ++i) {
            if (m > 0 && ent[lo + m - 1].c == ent[i].c) { ent[lo + m - 1].w += ent[i].w; continue; }
            ent[lo + m] = ent[i]; ++m;
        }
        rowlen[c + 1] = m;
    }
    out->n = k;
    out->rp = (int64_t*)malloc((size_t)(k + 1) * sizeof(int64_t));
    out->rp[0] = 0;
    for (int64_t c = 0; c < k; ++c) out->rp[c + 1] = out->rp[c] + rowlen[c + 1];
    out->col = (int32_t*)malloc((size_t)(out->rp[k] + 1) * sizeof(int32_t));
    out->w = (int64_t*)malloc((size_t)(out->rp[k] + 1) * sizeof(int64_t));
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t c = 0; c < k; ++c)
        for (int64_t i = 0; i < rowlen[c + 1]; ++i) {
            out->col[out->rp[c] + i] = ent[cnt[c] + i].c;
            out->w[out->rp[c] + i] = ent[cnt[c] + i].w;
        }
    free(cnt); free(ent); free(cur); free(rowlen);
}

/* ------------------------------------------------------------ Louvain */
/*
 * oracle_louvain: full multi-level run.
 *   prune      : pruning strategy deciding the active set of every iteration
 *                (§3.2-3.3):
 *                0 = none (baseline, every vertex evaluated)
 *                1 = MG, modularity-gain based (Eq. 6/7)
 *                2 = SM, strict movement based: v inactive iff neither
 *                    C[v] nor any C[u], u in N(v), gained or lost a member in
 *                    the previous iteration (reading c20)
 *                3 = RM, relaxed movement based: v active iff some
 *                    neighbour u != v changed community in the previous
 *                    iteration (reading c21)
 *                4 = MG+RM: inactive iff MG or RM says inactive
 *                SM and RM have no previous iteration in the first iteration of
 *                a level: every vertex is active there.
 *   check      : also evaluate pruned vertices and count those that would have
 *                moved (false negatives, Eq. 3 / P:147) and the active vertices
 *                that stay (false positives); pruned vertices still stay
 *   trace      : 0 none, 1 per-iteration records, 2 records + label snapshots,
 *                3 also the per-vertex inactive flags of every iteration
 *   max_iters  : per-level iteration cap (0 = none; honoured identically by the library)
 * Returns an opaque result (free with oracle_free).  status != 0 on error.
 */
void* oracle_louvain(int64_t n, const int64_t* row_ptr, const int32_t* col, const int64_t* w,
                     double gamma, double tol, int32_t max_levels, int32_t max_iters,
                     int prune, int check, int trace) {
    orc_result* R = (orc_result*)calloc(1, sizeof(orc_result));
    R->n0 = n;
    oracle_gamma_pq(gamma, &R->p, &R->q);
    int64_t p = R->p, q = R->q;
    if (n < 0 || n >= ((int64_t)1 << 31)) { R->status = 1; R->n0 = 0; return R; }
    int32_t* lab = (int32_t*)malloc((size_t)(n + 1) * sizeof(int32_t));
    for (int64_t v = 0; v < n; ++v) lab[v] = (int32_t)v;
    R->lab = lab;
    R->k = n;
    if (!(tol > 0) || p <= 0 || prune < 0 || prune > 4) { R->status = 1; return R; }
    int64_t nnz = row_ptr[n];
    /* level-0 graph (copied; unit weights materialised) */
    ograph G;
    G.n = n;
    G.rp = (int64_t*)malloc((size_t)(n + 1) * sizeof(int64_t));
    memcpy(G.rp, row_ptr, (size_t)(n + 1) * sizeof(int64_t));
    G.col = (int32_t*)malloc((size_t)(nnz + 1) * sizeof(int32_t));
    G.w = (int64_t*)malloc((size_t)(nnz + 1) * sizeof(int64_t));
    memcpy(G.col, col, (size_t)nnz * sizeof(int32_t));
    int64_t W = 0, maxd = 0;
    for (int64_t v = 0; v < n; ++v) {
        if (row_ptr[v + 1] < row_ptr[v]) { R->status = 1; break; }
        int64_t dv = 0;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            G.w[e] = w ? w[e] : 1;
            if (G.w[e] <= 0 || col[e] < 0 || col[e] >= n) { R->status = 1; break; }
            dv += G.w[e];
        }
        W += dv;
        if (dv > maxd) maxd = dv;
    }
    R->W = W;
    /* overflow budget: |scores| <= q*W*maxd must stay well inside __int128 */
    if (row_ptr[0] != 0) R->status = 1;
    /* overflow budget (include/gala.h GALA_E_OVERFLOW): max(p,q) * W^2 < 2^125 keeps every
       score, stay, Eq. 6 left-hand side and numerator N inside __int128 */
    (void)maxd;
    if (!R->status && (long double)(p > q ? p : q) * (long double)W * (long double)W >= 0x1p125L) R->status = 2;
    if (R->status || W == 0) {   /* reading c18: no edges -> singletons, Q := 0 */
        R->N = 0;
        free(G.rp); free(G.col); free(G.w);
        return R;
    }
    /* theta test (reading c7): dN < T with T = ceil(tol * q * W^2) in long double */
    i128 thr = (i128)ceill((long double)tol * (long double)q * (long double)W * (long double)W);

    for (int32_t level = 0;; ++level) {
        int64_t nl = G.n;
        int64_t* d = (int64_t*)calloc((size_t)nl, sizeof(int64_t));
        int64_t* s = (int64_t*)calloc((size_t)nl, sizeof(int64_t));
        int64_t* dp = (int64_t*)calloc((size_t)nl, sizeof(int64_t));
        int64_t* Sig = (int64_t*)calloc((size_t)nl, sizeof(int64_t));
        int32_t* size = (int32_t*)calloc((size_t)nl, sizeof(int32_t));
        int32_t* C = (int32_t*)malloc((size_t)nl * sizeof(int32_t));
        int32_t* nextC = (int32_t*)malloc((size_t)nl * sizeof(int32_t));
        /* movement history of the previous iteration (SM / RM strategies) */
        char* moved_prev = (char*)calloc((size_t)nl, 1);     /* v changed community */
        char* changed_prev = (char*)calloc((size_t)nl, 1);   /* community c gained or lost a member */
        int64_t maxdeg = 0;
        /* level init: every vertex its own community */
        for (int64_t v = 0; v < nl; ++v) {
            for (int64_t e = G.rp[v]; e < G.rp[v + 1]; ++e) {
                d[v] += G.w[e];
                if (G.col[e] == v) s[v] += G.w[e];
            }
            if (G.rp[v + 1] - G.rp[v] > maxdeg) maxdeg = G.rp[v + 1] - G.rp[v];
            C[v] = (int32_t)v; Sig[v] = d[v]; size[v] = 1; dp[v] = 0;
        }
        i128 N = 0;
        {
            i128 sd2 = 0; int64_t ss = 0;
            for (int64_t v = 0; v < nl; ++v) { sd2 += (i128)d[v] * d[v]; ss += s[v]; }
            N = (i128)q * W * ss - (i128)p * sd2;
        }
        i128 N_start = N;
        int nt = omp_get_max_threads();
        cw_pair** bufs = (cw_pair**)malloc((size_t)nt * sizeof(cw_pair*));
        for (int t = 0; t < nt; ++t) bufs[t] = (cw_pair*)malloc((size_t)(maxdeg + 1) * sizeof(cw_pair));
        int64_t iters = 0;
        for (int32_t it = 0;; ++it) {
            /* min over non-empty communities (reading c3) */
            int64_t minSig = INT64_MAX;
            for (int64_t c = 0; c < nl; ++c) if (Sig[c] > 0 && Sig[c] < minSig) minSig = Sig[c];
            int64_t n_active = 0, n_pruned = 0, n_fn = 0, n_fp = 0, bad = 0;
            unsigned char* pflag = trace >= 3 ? (unsigned char*)calloc((size_t)nl + 1, 1) : NULL;
            /* Alg. 1 lines 3-4: every vertex decides from the start-of-iteration state */
            #pragma omp parallel for schedule(dynamic, 256) reduction(+:n_active, n_pruned, n_fn, n_fp, bad)
            for (int64_t v = 0; v < nl; ++v) {
                nextC[v] = C[v];
                if (d[v] == 0) continue;
                int pruned = 0;
                if (prune == 1 || prune == 4) {
                    /* Eq. 6 multiplied by q*W:  q W (2 d' - d) + p (minSig - Sig[C[v]]) d >= 0 */
                    i128 lhs = (i128)q * W * (2 * dp[v] - d[v]) + (i128)p * (minSig - Sig[C[v]]) * d[v];
                    pruned = lhs >= 0;
                }
                if (prune == 2 && it > 0) {   /* SM: every community around v unchanged */
                    int chg = changed_prev[C[v]];
                    for (int64_t e = G.rp[v]; e < G.rp[v + 1] && !chg; ++e)
                        if (changed_prev[C[G.col[e]]]) chg = 1;
                    pruned = !chg;
                }
                if ((prune == 3 || prune == 4) && it > 0) {   /* RM: no neighbour moved */
                    int nb_moved = 0;
                    for (int64_t e = G.rp[v]; e < G.rp[v + 1] && !nb_moved; ++e)
                        if (G.col[e] != v && moved_prev[G.col[e]]) nb_moved = 1;
                    if (!nb_moved) pruned = 1;   /* MG+RM: pruned by either rule */
                }
                if (pruned && pflag) pflag[v] = 1;
                if (pruned && !check) { n_pruned++; continue; }
                int64_t d_own = 0;
                int32_t b = decide(&G, v, C, Sig, size, d, dp, W, p, q, bufs[omp_get_thread_num()], &d_own);
                if (d_own != dp[v]) bad++;                  /* maintained d' must equal its definition */
                if (pruned) { n_pruned++; if (b != C[v]) n_fn++; continue; }
                n_active++;
                if (b == C[v]) n_fp++;
                nextC[v] = b;
            }
            if (bad) R->status = 3;
            /* Alg. 1 line 5: update the community set (Sigma_tot = D_V, sizes) */
            int64_t n_moved = 0;
            memset(moved_prev, 0, (size_t)nl);
            memset(changed_prev, 0, (size_t)nl);
            for (int64_t v = 0; v < nl; ++v) {
                if (nextC[v] == C[v]) continue;
                moved_prev[v] = 1;
                changed_prev[C[v]] = 1;
                changed_prev[nextC[v]] = 1;
                Sig[C[v]] -= d[v]; size[C[v]]--;
                Sig[nextC[v]] += d[v]; size[nextC[v]]++;
                C[v] = nextC[v];
                n_moved++;
            }
            /* Alg. 1 lines 6-7: d_{C[v]}(v) from its definition (self loop excluded) */
            #pragma omp parallel for schedule(dynamic, 256)
            for (int64_t v = 0; v < nl; ++v) {
                int64_t x = 0;
                for (int64_t e = G.rp[v]; e < G.rp[v + 1]; ++e)
                    if (G.col[e] != v && C[G.col[e]] == C[v]) x += G.w[e];
                dp[v] = x;
            }
            /* Alg. 1 lines 8-11: D_C, D_V, next_Q (Eq. 1) */
            int64_t sumDC = 0;
            for (int64_t v = 0; v < nl; ++v) sumDC += dp[v] + s[v];
            i128 S2 = 0;
            for (int64_t c = 0; c < nl; ++c) S2 += (i128)Sig[c] * Sig[c];
            i128 Nn = (i128)q * W * sumDC - (i128)p * S2;
            ++iters;
            if (trace) {
                orc_rec x;
                x.level = level; x.iter = it; x.n_level = nl;
                x.n_active = n_active; x.n_pruned = n_pruned; x.n_moved = n_moved; x.n_fn = n_fn;
                x.n_fp = check ? n_fp : 0;
                x.N = Nn; x.labels = NULL; x.pruned = pflag; pflag = NULL;
                if (trace >= 2) {
                    x.labels = (int32_t*)malloc((size_t)nl * sizeof(int32_t));
                    memcpy(x.labels, C, (size_t)nl * sizeof(int32_t));
                }
                push_rec(R, x);
            }
            free(pflag);
            /* Alg. 1 lines 12-13: Delta Q < theta (moves of this iteration are kept, c6) */
            int converged = (n_moved == 0) || (Nn - N < thr);
            N = Nn;
            if (converged || (max_iters > 0 && it + 1 >= max_iters)) break;
        }
        for (int t = 0; t < nt; ++t) free(bufs[t]);
        free(bufs);
        /* phase 2 relabel: non-empty communities in order of their smallest member (c9) */
        int32_t* minmem = (int32_t*)malloc((size_t)nl * sizeof(int32_t));
        for (int64_t c = 0; c < nl; ++c) minmem[c] = INT32_MAX;
        for (int64_t v = nl - 1; v >= 0; --v) minmem[C[v]] = (int32_t)v;
        int32_t* cnew = (int32_t*)malloc((size_t)nl * sizeof(int32_t));
        int64_t k = 0;
        for (int64_t v = 0; v < nl; ++v)
            if (minmem[C[v]] == v) cnew[C[v]] = (int32_t)k++;
        int32_t* newid = (int32_t*)malloc((size_t)nl * sizeof(int32_t));
        for (int64_t v = 0; v < nl; ++v) newid[v] = cnew[C[v]];
        for (int64_t v0 = 0; v0 < n; ++v0) lab[v0] = newid[lab[v0]];
        orc_level L = { nl, G.rp[nl], iters, N_start, N };
        push_lev(R, L);
        int stop = (k == nl) || (max_levels > 0 && level + 1 >= max_levels) ||
                   (N - N_start < thr);
        free(d); free(s); free(dp); free(Sig); free(size); free(C); free(nextC); free(minmem); free(cnew);
        free(moved_prev); free(changed_prev);
        if (stop) { free(newid); break; }
        ograph H;
        coarsen(&G, newid, k, &H);
        free(newid);
        free(G.rp); free(G.col); free(G.w);
        G = H;
    }
    free(G.rp); free(G.col); free(G.w);
    /* canonical ids 0..k-1 in order of smallest original member (c19) */
    {
        int32_t* first = (int32_t*)malloc((size_t)(n + 1) * sizeof(int32_t));
        for (int64_t c = 0; c < n; ++c) first[c] = -1;
        int32_t k = 0;
        for (int64_t v = 0; v < n; ++v) { if (first[lab[v]] < 0) first[lab[v]] = k++; lab[v] = first[lab[v]]; }
        R->k = k;
        free(first);
    }
    /* final Q re-verified on G0 from the labels */
    {
        ograph G0;
        G0.n = n; G0.rp = (int64_t*)row_ptr; G0.col = (int32_t*)col;
        G0.w = (int64_t*)malloc((size_t)(nnz + 1) * sizeof(int64_t));
        for (int64_t e = 0; e < nnz; ++e) G0.w[e] = w ? w[e] : 1;
        R->N = modularity_num(&G0, lab, W, p, q);
        free(G0.w);
    }
    return R;
}

/* ------------------------------------------------------------- accessors */
static void split128(i128 x, int64_t* hi, uint64_t* lo) { *hi = (int64_t)(x >> 64); *lo = (uint64_t)x; }

int oracle_status(void* h) { return ((orc_result*)h)->status; }
int64_t oracle_num_communities(void* h) { return ((orc_result*)h)->k; }
void oracle_labels(void* h, int32_t* out) {
    orc_result* R = (orc_result*)h;
    memcpy(out, R->lab, (size_t)R->n0 * sizeof(int32_t));
}
/* out[0]=W out[1]=p out[2]=q out[3]=N_hi out[4]=N_lo(bits) out[5]=#levels out[6]=#records */
void oracle_summary(void* h, int64_t* out) {
    orc_result* R = (orc_result*)h;
    uint64_t lo;
    out[0] = R->W; out[1] = R->p; out[2] = R->q;
    split128(R->N, &out[3], &lo); out[4] = (int64_t)lo;
    out[5] = R->nlev; out[6] = R->nrec;
}
double oracle_modularity(void* h) {
    orc_result* R = (orc_result*)h;
    if (R->W == 0) return 0.0;
    return (double)((long double)R->N / ((long double)R->q * (long double)R->W * (long double)R->W));
}
/* rec: level, iter, n_level, n_active, n_pruned, n_moved, n_fn, N_hi, N_lo, n_fp */
void oracle_record(void* h, int64_t i, int64_t* out) {
    orc_rec* x = &((orc_result*)h)->rec[i];
    uint64_t lo;
    out[0] = x->level; out[1] = x->iter; out[2] = x->n_level; out[3] = x->n_active;
    out[4] = x->n_pruned; out[5] = x->n_moved; out[6] = x->n_fn;
    split128(x->N, &out[7], &lo); out[8] = (int64_t)lo;
    out[9] = x->n_fp;
}
int oracle_record_labels(void* h, int64_t i, int32_t* out) {
    orc_rec* x = &((orc_result*)h)->rec[i];
    if (!x->labels) return 1;
    memcpy(out, x->labels, (size_t)x->n_level * sizeof(int32_t));
    return 0;
}
int oracle_record_pruned(void* h, int64_t i, unsigned char* out) {
    orc_rec* x = &((orc_result*)h)->rec[i];
    if (!x->pruned) return 1;
    memcpy(out, x->pruned, (size_t)x->n_level);
    return 0;
}
/* level: n, nnz, iters, Nstart_hi, Nstart_lo, Nend_hi, Nend_lo */
void oracle_level(void* h, int64_t i, int64_t* out) {
    orc_level* L = &((orc_result*)h)->lev[i];
    uint64_t lo;
    out[0] = L->n; out[1] = L->nnz; out[2] = L->iters;
    split128(L->N_start, &out[3], &lo); out[4] = (int64_t)lo;
    split128(L->N_end, &out[5], &lo); out[6] = (int64_t)lo;
}
void oracle_free(void* h) {
    orc_result* R = (orc_result*)h;
    if (!R) return;
    for (int64_t i = 0; i < R->nrec; ++i) { free(R->rec[i].labels); free(R->rec[i].pruned); }
    free(R->rec); free(R->lev); free(R->lab); free(R);
}

/*
 * oracle_partition_numerator: N of an arbitrary partition (Eq. 1 x q*W^2).
 * out[0]=W out[1]=N_hi out[2]=N_lo.  Returns 0, or 1 on invalid input.
 */
int oracle_partition_numerator(int64_t n, const int64_t* row_ptr, const int32_t* col, const int64_t* w,
                               const int32_t* labels, double gamma, int64_t* out) {
    int64_t p, q;
    oracle_gamma_pq(gamma, &p, &q);
    int64_t nnz = row_ptr[n];
    ograph G;
    G.n = n; G.rp = (int64_t*)row_ptr; G.col = (int32_t*)col;
    G.w = (int64_t*)malloc((size_t)(nnz + 1) * sizeof(int64_t));
    int64_t W = 0;
    for (int64_t e = 0; e < nnz; ++e) { G.w[e] = w ? w[e] : 1; W += G.w[e]; }
    for (int64_t v = 0; v < n; ++v) if (labels[v] < 0 || labels[v] >= n) { free(G.w); return 1; }
    i128 N = modularity_num(&G, labels, W, p, q);
    free(G.w);
    uint64_t lo;
    out[0] = W; split128(N, &out[1], &lo); out[2] = (int64_t)lo;
    return 0;
}

/*
 * oracle_move_gain: for partition `labels` (ids in [0,n)) and vertex v, the
 * closed-form 2*(score(target) - stay) of moving v to community `target`
 * (Eq. 2 with reading c1), computed from D_V/d sums of the given partition.
 * out[0]=hi out[1]=lo.  Used by the P2 pin against brute-force N differences.
 */
void oracle_move_gain(int64_t n, const int64_t* row_ptr, const int32_t* col, const int64_t* w,
                      const int32_t* labels, double gamma, int64_t v, int32_t target, int64_t* out) {
    int64_t p, q;
    oracle_gamma_pq(gamma, &p, &q);
    int64_t W = 0;
    int64_t* Sig = (int64_t*)calloc((size_t)n, sizeof(int64_t));
    for (int64_t x = 0; x < n; ++x)
        for (int64_t e = row_ptr[x]; e < row_ptr[x + 1]; ++e) {
            int64_t ww = w ? w[e] : 1;
            W += ww; Sig[labels[x]] += ww;
        }
    int64_t dv = 0, dp = 0, wt = 0;
    for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
        int64_t ww = w ? w[e] : 1;
        dv += ww;
        if (col[e] == v) continue;
        if (labels[col[e]] == labels[v]) dp += ww;
        if (labels[col[e]] == target) wt += ww;
    }
    i128 stay = (i128)q * W * dp - (i128)p * (Sig[labels[v]] - dv) * dv;
    i128 sc = (i128)q * W * wt - (i128)p * Sig[target] * dv;
    if (target == labels[v]) sc = stay;
    i128 g2 = 2 * (sc - stay);
    free(Sig);
    uint64_t lo;
    split128(g2, &out[0], &lo); out[1] = (int64_t)lo;
}
