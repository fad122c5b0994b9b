/*
 * gala.h — C ABI of the B200-native GALA Louvain library (libgala.so).
 *
 * GALA = "Swift Unfolding of Communities: GPU-Accelerated Louvain Algorithm",
 * Wang et al., PPoPP'25.  "P:N" = line N of the paper text.
 *
 * The library computes a community assignment of an undirected graph with
 * positive integer edge weights that greedily maximises modularity (Eq. 1,
 * P:96-101) with the multi-level Louvain method: phase 1 is the BSP
 * local-moving iteration of Alg. 1 with MG pruning (Eq. 6/7,
 * P:197-203) and delta community-weight updating (§3.5); phase 2
 * compresses communities into super vertices.  Every step runs in
 * hand-written sm_100a CUDA kernels on the device the graph lives on.
 *
 * Conventions:
 *  - Graph input is a symmetric CSR: for every entry (v,u,w) the entry
 *    (u,v,w) exists.  A self loop (v,v,w) is stored ONCE and counts once in
 *    d(v) and in D_C.  Duplicate entries are allowed and summed.
 *  - Weights are positive integers (int64).  NULL weights = all 1.
 *  - gamma (resolution) is quantised to p/q = round(gamma*2^16)/2^16.
 *    All gains and modularity numerators are exact integers; decisions are
 *    bit-for-bit reproducible and independent of thread/block/GPU counts.
 *  - Ties go to the lowest community id; Grappolo singleton swap suppression
 *    (P:141 footnote 1); a vertex moves only if its best gain beats staying.
 *  - Convergence: the iteration (and the level loop) stops when the exact
 *    numerator gain dN = N' - N < T with T = ceil(tol * q * W^2) evaluated in
 *    x87 long double (Alg. 1 lines 12-13, theta = tol, P:340 uses 1e-6).
 *
 * Ownership: input arrays are copied; the caller may free them on return.
 * Outputs are written into caller buffers.  The handle owns all device memory
 * and frees it in gala_graph_free.  Every call returns a gala_status; no C++
 * exception crosses this boundary.  On error gala_last_error() returns a
 * thread-local message.  Calls on one handle must not run concurrently.
 */
#ifndef GALA_H
#define GALA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gala_graph_s* gala_graph;

typedef enum {
    GALA_OK = 0,
    GALA_E_INVALID = 1,   /* malformed CSR, weight <= 0, n >= 2^31, bad option/argument */
    GALA_E_OVERFLOW = 2,  /* max(p,q) * W^2 >= 2^125: exact integer gains would overflow */
    GALA_E_NOMEM = 3,     /* device allocation failed */
    GALA_E_CUDA = 4,      /* CUDA runtime error (message in gala_last_error) */
    GALA_E_NCCL = 5,      /* NCCL error or NCCL unavailable (multi-GPU only) */
    GALA_E_STATE = 6      /* call not valid in this state (e.g. results before gala_run) */
} gala_status;

/* Library version string (static storage). */
const char* gala_version(void);

/* Thread-local message of the last non-OK status (static until the next call). */
const char* gala_last_error(void);

/*
 * gala_graph_from_csr — build a handle from a HOST CSR (problem statement,
 * §2.1: G = {V, E, w}).
 *   n        : number of vertices, 0 <= n < 2^31
 *   row_ptr  : host int64[n+1], row_ptr[0] = 0, non-decreasing
 *   col_idx  : host int32[row_ptr[n]], each in [0, n)
 *   weights  : host int64[row_ptr[n]] each > 0, or NULL (all 1)
 *   device   : CUDA device ordinal the graph and all kernels live on
 *   stream   : cudaStream_t as an integer (0 = the library's own stream)
 *   out      : receives the handle
 * Copies the graph to the device (H2D) and validates it.  Symmetry is NOT
 * checked unless option "check_symmetric" is set afterwards and
 * gala_validate is called.
 */
gala_status gala_graph_from_csr(int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                                const int64_t* weights, int device, uintptr_t stream,
                                gala_graph* out);

/*
 * gala_graph_from_csr_device — same, but row_ptr/col_idx/weights are DEVICE
 * pointers on `device` (e.g. torch CUDA tensors).  The data is copied
 * device-to-device; the caller keeps ownership of its buffers.
 */
gala_status gala_graph_from_csr_device(int64_t n, const int64_t* d_row_ptr, const int32_t* d_col_idx,
                                       const int64_t* d_weights, int device, uintptr_t stream,
                                       gala_graph* out);

/* Verify symmetry of the stored CSR (O(nnz log) device check). GALA_E_INVALID if not. */
gala_status gala_validate(gala_graph g);

/*
 * gala_run — full multi-level Louvain: phase 1 (Alg. 1) to
 * convergence, then phase 2 coarsening, repeated until no community merges,
 * the level's numerator gain is below T, or max_levels levels ran.
 *   gamma      : resolution (> 0), quantised as above
 *   tol        : theta > 0 (P:340 uses 1e-6)
 *   max_levels : <= 0 means until converged
 * Always restarts from singletons; deterministic.  Synchronises the
 * handle's stream before returning.
 */
gala_status gala_run(gala_graph g, double gamma, double tol, int32_t max_levels);

/*
 * gala_get_communities — final labels of the level-0 vertices, canonical ids
 * 0..k-1 in order of each community's smallest vertex id.
 *   labels : host int32[n]; n must equal the graph's n
 *   num_communities : optional (nullable) receives k
 */
gala_status gala_get_communities(gala_graph g, int32_t* labels, int64_t n, int64_t* num_communities);

/* Same as gala_get_communities but writes into a DEVICE buffer on the graph's device. */
gala_status gala_get_communities_device(gala_graph g, int32_t* d_labels, int64_t n,
                                        int64_t* num_communities);

/*
 * gala_modularity — Q_gamma (Eq. 1 with resolution) of the final partition,
 * recomputed exactly on the level-0 graph and rounded once to double.
 */
gala_status gala_modularity(gala_graph g, double* q);

/*
 * gala_modularity_numerator — exact N = q*W*sum_C D_C(C) - p*sum_C D_V(C)^2
 * of the final partition as a 128-bit two's-complement (hi, lo) pair, plus W,
 * p and q.  Q = N / (q W^2).  Any out pointer may be NULL.
 */
gala_status gala_modularity_numerator(gala_graph g, int64_t* n_hi, uint64_t* n_lo, int64_t* W,
                                      int64_t* p, int64_t* q);

/* Free the handle and all its device memory.  NULL is a no-op.  The handle's (synchronised,
 * idle) memory pool of the default allocator is parked per device and adopted by the next
 * handle created on that device, so create/run/free cycles do not map fresh pages every time;
 * at most one pool per device is kept (multi-GPU handles and user-allocator blocks are always
 * released). */
void gala_graph_free(gala_graph g);

/*
 * gala_set_option — tuning / test hooks.  Options never change results
 * (labels are identical for every setting) except "max_iters" (a per-level
 * iteration cap honoured identically by the oracle) and "prune" (pruning
 * changes which vertices are evaluated; the oracle takes the same flag).
 *   "prune"          pruning strategy of the active set (§3.2-3.3), default 1:
 *                    0 none (baseline), 1 MG modularity-gain based (Eq. 6/7, lossless),
 *                    2 SM strict movement based (lossless), 3 RM relaxed movement
 *                    based (lossy), 4 MG+RM (lossy, same moves as RM).
 *                    SM / RM see the moves of the previous iteration of the level
 *                    (readings c20 / c21).  2-4 are single-GPU only.
 *   "prune_check"    0/1   instrument the pruning: pruned vertices are evaluated too but
 *                          never moved; per iteration the trace counts false negatives
 *                          (pruned, would have moved) and false positives (active, stayed),
 *                          Eq. 3 / P:145-147.  Results are unchanged.
 *   "trace"          0/1/2 per-iteration records; 2 also copies labels each iteration
 *   "check"          0/1   debug: verify maintained d'(v) against its definition
 *   "timing"         0/1   per-kernel CUDA-event timing (gala_get_kernel_stats)
 *   "max_iters"      >= 0  per-level iteration cap (0 = none)
 *   "bin_sub4" "bin_sub8" "bin_sub16" "bin_sub32" "bin_warp" "bin_warp512" "bin_block"
 *                    row-length upper bounds of the dispatch bins (non-decreasing;
 *                    each <= 4, 8, 16, 32, 128, 512, 2^30 respectively; defaults
 *                    4 8 16 32 128 512 16384).  Rows longer than "bin_block" take the
 *                    multi-block hub path (chunks of 1024 entries over all SMs).
 *   "delta_update"   0 = always recompute d', 1 = always delta, 2 = adaptive (default)
 *   "delta_den"      [1, 64] adaptive rule: delta iff the moved vertices' row entries are
 *                          <= nnz / delta_den (default 2)
 *   "force_i128"     0/1   use the 128-bit gain path even when 64-bit suffices
 *   "force_wide"     0/1/2 1: unpacked 64-bit gains everywhere (no packed keys); 2: the level runs
 *                          as if it needed them but the short-row bins may still pack (bin_packed)
 *   "bin_packed"     0/1   on a level whose hubs need unpacked (score, c) keys, the bins of rows
 *                          <= bin_warp512 still use packed keys when max(p,q) W row 2^idbits < 2^62
 *                          (default 1; unit-weight levels only)
 *   "singleton"      0/1   first iteration of a level via the singleton fast path (default 1)
 *   "ckey"           0/1   keep a per-entry copy of C[col] on level 0, maintained by the delta
 *                          update (default 0; trades nnz*4 bytes for one gather per entry)
 *   "hub_smem_slots" power of two in [64, 16384], shared-memory slots of the block hash table (default 8192)
 *   "cuda_graph"     0/1   run each level's iterations as a conditional CUDA graph (default 1)
 *   "concurrent"     0/1   run the degree bins' decide kernels as parallel branches on side
 *                          streams (default 0: measured slower on B200 -- the bins contend for L2 and smem; off whenever "timing" is on)
 *   "log_cap"        device iteration-log capacity (default 4096)
 *   "sync_mode"      multi-GPU label exchange: 0 adaptive (default), 1 dense, 2 sparse (host
 *                          backend; the fabric sends sparse whenever the list fits, 2 = 0 there)
 *   "dist_backend"   multi-GPU iteration: 0 fabric (default; device-resident over peer memory,
 *                          no host round trip per iteration, CUDA-graph captured, delta d' via the
 *                          mirror block, send-to-owner phase 2), 1 host-driven collectives (one
 *                          host round trip per iteration, d' recomputed, phase 2 all-gathered)
 *   "verbose"        0/1   host-side phase timings on stderr
 *   "block_split"    block bin split point (default 1024; 0: one class): on levels with rows longer
 *                          than it, rows <= split run in 256-thread blocks with a small arena, the
 *                          rest in the 512-thread full-arena kernel
 *   "agg_big_chunk"  0/1   phase 2: big communities in 4096-entry chunks over the whole GPU with a
 *                          block-smem pre-combine (default 1); 0: 32 blocks per big community
 *   "agg_bound"      0/1   phase 2: big-community global tables sized from the chunks' distinct counts
 *                          (two passes, default 1) instead of from min(entries, k)
 *   "agg_chunk"      [1, 4096] entries per big-community chunk (test hook, default 4096)
 *   "agg_big_ent"    >= 1  phase 2: communities with more entries than this take the chunked big
 *                          path even when their table fits in shared memory (default 32768: one
 *                          block per huge community serialised the Orkut level-0 coarsening)
 *   "agg_scap"       [512, 8192] largest phase-2 shared-memory table; communities needing more
 *                          slots take the big (global-table) path (test hook, default 8192)
 */
gala_status gala_set_option(gala_graph g, const char* key, int64_t value);

/*
 * gala_set_allocator — device-memory hook (SURVEY.md §8(b) "allocator hook").  Process-wide;
 * applies to every block any handle allocates AFTER the call (a block is always returned to the
 * allocator that made it).  alloc(bytes, device, stream, ctx) returns a device pointer valid for
 * work ordered on `stream` (NULL -> GALA_E_NOMEM from the call that needed it);
 * free(ptr, bytes, device, stream, ctx) may recycle it for later work on that stream.
 * Both NULL restores the default (a per-handle stream-ordered cudaMemPool); exactly one NULL is
 * GALA_E_INVALID.  The Python binding routes it to torch.cuda's caching allocator
 * (gala.use_torch_allocator()).  Allocation happens per level, so callback cost is immaterial.
 */
typedef void* (*gala_alloc_fn)(size_t bytes, int device, uintptr_t stream, void* ctx);
typedef void (*gala_free_fn)(void* ptr, size_t bytes, int device, uintptr_t stream, void* ctx);
gala_status gala_set_allocator(gala_alloc_fn alloc_fn, gala_free_fn free_fn, void* ctx);

/*
 * gala_get_stats — JSON object with per-level and per-iteration statistics
 * of the last gala_run (levels, iterations, active/pruned/moved counts,
 * edges scanned, timings).  Writes at most cap bytes including the NUL;
 * returns GALA_E_INVALID if cap is too small (required size in *needed).
 */
gala_status gala_get_stats(gala_graph g, char* json_buf, int64_t cap, int64_t* needed);

/*
 * Trace access (option "trace" >= 1).  Record i (0 <= i < count) is
 * int64[16]: level, iter, n_level, n_active, n_pruned, n_moved,
 *            N_hi, N_lo (numerator after the iteration), edges_scanned
 *            (sum of deg(v) over the active vertices), distinct_communities_seen,
 *            delta_update_used, sync (multi-GPU fabric: 1 + senders that exchanged their
 *            whole label slice; 0 otherwise), n_false_negative (option "prune_check"),
 *            n_false_positive ("prune_check"; multi-GPU fabric: bytes this rank received),
 *            iteration device time in ns (%globaltimer, reduction to reduction),
 *            algorithmic bytes of the iteration (single GPU).
 * Labels (trace == 2): level-local community of every level vertex after
 * the iteration; out must hold n_level entries.
 */
gala_status gala_get_trace_count(gala_graph g, int64_t* count);
gala_status gala_get_trace_record(gala_graph g, int64_t i, int64_t* out16);
gala_status gala_get_trace_labels(gala_graph g, int64_t i, int32_t* out, int64_t n_level);

/*
 * Per-kernel-class device time of the last gala_run (option "timing").
 * For class k (0 <= k < *count): name (static string), launches, total
 * milliseconds, algorithmic bytes.
 */
gala_status gala_get_kernel_stats(gala_graph g, int32_t k, const char** name, int64_t* launches,
                                  double* ms, double* alg_bytes, int32_t* count);

/* ---------------------------------------------------------------- multi-GPU
 * 1D vertex partition, one process per GPU (§4.3).  Rank r owns
 * the contiguous vertex range [v_begin, v_end) and its CSR rows (global
 * column ids).  Community state (C, Sigma_tot, size, d) is replicated.  After
 * every iteration each rank's moves reach every replica, densely (its whole
 * label slice) or sparsely ((vertex, community) pairs), chosen per sender by
 * bytes; every replica then applies the same moves, so Sigma_tot
 * needs no all-reduce (the zero-communication equivalent of SURVEY.md §8(e)).
 * Default backend ("dist_backend" 0): the exchange, two device-side barriers and
 * the counter sums run in kernels over peer memory (CUDA IPC mappings set up
 * once over NCCL), so an iteration has no host round trip.  Backend 1 issues
 * NCCL collectives from the host.  Results are identical to 1 GPU.
 */

/* 128-byte ncclUniqueId for rank 0 to broadcast (GALA_E_NCCL if NCCL cannot be loaded). */
gala_status gala_nccl_unique_id(void* out128);

/*
 * gala_loopback_unique_id — TEST HOOK: a uid that makes gala_graph_from_csr_dist
 * run `world` ranks as threads of ONE process on one device (device-to-device
 * copies + host barriers instead of NCCL), so the partitioned algorithm can be
 * exercised where only one GPU exists.  Never used by the product path.
 */
gala_status gala_loopback_unique_id(void* out128);

/*
 * gala_graph_from_csr_dist — collective over `world` ranks.
 *   uid128      : the same ncclUniqueId on every rank
 *   n_global    : global vertex count
 *   v_begin/end : owned vertex range (ranges tile [0, n_global) in rank order)
 *   local_row_ptr : host int64[v_end - v_begin + 1], local_row_ptr[0] = 0
 *   col_idx     : host int32[local nnz], GLOBAL vertex ids
 *   weights     : host int64[local nnz] or NULL
 * The NCCL communicator is created on the first call with a given uid and
 * cached for the life of the process; later handles built with the same uid
 * (on the same ranks) reuse it.
 */
gala_status gala_graph_from_csr_dist(const void* uid128, int rank, int world, int device,
                                     int64_t n_global, int64_t v_begin, int64_t v_end,
                                     const int64_t* local_row_ptr, const int32_t* col_idx,
                                     const int64_t* weights, uintptr_t stream, gala_graph* out);

/*
 * gala_nmi_device — normalised mutual information of two partitions (quality report of
 * Table 4; definition of ref. [52], Strehl & Ghosh 2002):
 *   NMI = I(X;Y) / sqrt(H(X) H(Y)),  I = sum_ab (n_ab/n) ln(n n_ab / (n_a n_b)),
 *   H(X) = -sum_a (n_a/n) ln(n_a/n);  1 if both partitions have one cluster, 0 if only one has.
 *   d_x, d_y : DEVICE int32[n] on `device`, labels in [0, n) (e.g. gala_get_communities_device
 *              output and an LFR planted partition); read only, caller keeps ownership
 *   n        : 0 <= n < 2^31 (n = 0 gives 1)
 *   stream   : cudaStream_t as an integer (0 = legacy default stream); synchronised on return
 *   out      : receives the NMI (fp64; contingency counts are exact integers, the three log
 *              sums are reduced in a fixed order, so the value is reproducible)
 * GALA_E_INVALID for a null pointer, n out of range or a label outside [0, n); GALA_E_CUDA on
 * a device error.  Not a step of the Louvain path: it reports the quality of a result.
 */
gala_status gala_nmi_device(const int32_t* d_x, const int32_t* d_y, int64_t n, int device, uintptr_t stream,
                            double* out);

/*
 * gala_partition_ranges — host-only helper: edge-balanced contiguous split of
 * n vertices over `world` ranks (each range's entry count ~ nnz/world).
 * bounds: int64[world+1].
 */
gala_status gala_partition_ranges(int64_t n, const int64_t* row_ptr, int world, int64_t* bounds);

#ifdef __cplusplus
}
#endif

#endif /* GALA_H */
