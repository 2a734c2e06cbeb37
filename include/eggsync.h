/*
 * eggsync.h -- C ABI of the B200-native EGG-SynC synchronization update.
 *
 * Paper: J. R. Jorgensen, I. Assent, "EGG-SynC: Exact GPU-parallelized
 * Grid-based Clustering by Synchronization", EDBT 2023.  Citations "L<n>"
 * are lines of that paper's text with the section / equation /
 * algorithm they fall in.
 *
 * Problem statement (L66-L70 §3, Def 4.1): given D in [0,1]^{n x d}
 * and a radius eps, iterate the Kuramoto update (Eq.1)
 *     p_i <- p_i + 1/|N_eps(p)| * sum_{q in N_eps(p)} sin(q_i - p_i),
 *     N_eps(p) = {q : ||p - q|| <= eps}  (p itself included, L66)
 * synchronously until the synchronization criterion (Def 4.2)
 * holds, then return the clusters: the non-empty grid cells of width
 * eps/(2 sqrt d) (gatherCluster, L256; cell width L252).
 *
 * Conventions shared by every entry point
 *  - All functions have C linkage, are reentrant with respect to distinct
 *    buffers, and never throw across the ABI.
 *  - Ownership: the caller owns every buffer passed in.  The library
 *    allocates its device workspace per call (or per context), reuses it
 *    across iterations (as the paper does, L195) and frees it before
 *    returning (or in eggsync_ctx_destroy).
 *  - Validation happens before any output is written: on EGGSYNC_EINVAL or
 *    EGGSYNC_EDOMAIN every output buffer is left untouched.  After
 *    EGGSYNC_ENOMEM / EGGSYNC_ECUDA outputs are unspecified.
 *  - eps is used exactly as the given float; every derived constant
 *    (eps^2, c_w, 1/c_w, w, delta) is computed in fp64 from (double)eps.
 *  - Arithmetic: coordinates are float32; neighbour sums are accumulated in
 *    fp32 chunks flushed into fp64; cell / subtree summaries are exact
 *    64-bit fixed-point sums of fp64 sin/cos; the update epilogue is fp64.
 *    The eps-predicate is decided in fp32 with a proven error band; pairs
 *    inside the band are re-decided in fp64 exactly as sum_i (q_i - p_i)^2
 *    <= eps^2 (dimension order, no FMA).
 *  - There is no CPU fallback: without a usable CUDA device every compute
 *    entry point returns EGGSYNC_ECUDA.
 */
#ifndef EGGSYNC_H
#define EGGSYNC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define EGGSYNC_OK 0
#define EGGSYNC_NOT_CONVERGED 1 /* max_iters reached: outputs hold the last state, labels = its cells */
#define EGGSYNC_EINVAL (-1)     /* NULL pointer, n < 1 or n > INT32_MAX, d < 1 or d > EGGSYNC_MAX_D,
                                   eps not finite or <= 0, grid too fine (d*ceil(log2 w) > 512 bits) */
#define EGGSYNC_EDOMAIN (-2)    /* a coordinate is NaN/Inf or outside [0,1] (L70, L290, L354) */
#define EGGSYNC_ENOMEM (-3)     /* device allocation failed */
#define EGGSYNC_ECUDA (-4)      /* CUDA error or no device; details in eggsync_last_error() */
#define EGGSYNC_ENCCL (-5)      /* reserved: collective failure (multi-GPU driver) */

#define EGGSYNC_MAX_D 32

/* termination modes (ambiguity register R1/F3 in DESIGN.md) */
#define EGGSYNC_TERM_GRID 0 /* first term via |cell(p)| == |N_eps(p)| (Alg 3 l.14-15 L248, L252) */
#define EGGSYNC_TERM_DEF42 1 /* Def 4.2 literally (L106-110): term (i) "no pair with eps/2 < ||p-q|| <= eps",
                                term (ii) with MBR(N_{eps/2}(q)); labels = connected components of
                                the eps-graph of the returned state (Theorem 4.7).  eggsync_cluster_ex
                                only; the grid update, the terms and the labels evaluated on the
                                grid's radix tree (work proportional to the neighbourhoods, F3). */
#define EGGSYNC_TERM_DEF42_DIRECT 2 /* the same criterion and labels on the direct (all-pairs,
                                O(n^2 d) per iteration) kernels of eggsync_sync_step, not the grid:
                                a second implementation for cross-checks; on opts.stream (NULL:
                                the legacy default stream); ignores cw_factor and stats other
                                than iters. */

/*
 * Per-stage timings of the last call, mirroring the columns of Table 1
 * (L364-371): allocating, build structure, update, extra check,
 * clustering, free.  Seconds, measured with CUDA events on the call's
 * stream.  Work counters are summed over iterations.
 */
typedef struct eggsync_stats {
  double t_alloc, t_build, t_update, t_extra_check, t_cluster, t_free, t_transfer;
  int32_t iters;
  int32_t n_cells_first, n_cells_last;
  int32_t sort_skipped; /* iterations whose keys were already sorted */
  int64_t device_bytes; /* workspace high-water mark */
} eggsync_stats;

typedef struct eggsync_opts {
  int32_t struct_size;     /* sizeof(eggsync_opts); ABI versioning */
  int32_t max_iters;       /* default 10000 (L306: "a maximum number of iterations could be used") */
  int32_t device;          /* CUDA ordinal; -1 = current device */
  int32_t device_pointers; /* 1: points / labels / coords_out / nbr_count_out are device pointers */
  void *stream;            /* cudaStream_t to run on; NULL = library-owned stream */
  int32_t term_mode;       /* EGGSYNC_TERM_GRID (default), _DEF42 or _DEF42_DIRECT (cluster_ex only) */
  float *coords_out;       /* optional n*d row-major final coordinates (original point order) */
  int32_t *nbr_count_out;  /* optional, step only: |N_eps(p)| on D^t, original order */
  eggsync_stats *stats;    /* optional */
  double cw_factor;        /* grid cell width c_w = cw_factor * eps / (2 sqrt d); (0, 1], default 1.
                              L252 only requires c_w <= sqrt((eps/2)^2 / d): any smaller width keeps
                              the grid first term equivalent to Def 4.2 term (i) and Theorem 4.7's
                              labels; smaller cells make the criterion stricter (never earlier).
                              Outside (0, 1] -> EGGSYNC_EINVAL. */
} eggsync_opts;

/* Fill *o with the defaults above (struct_size set). */
void eggsync_default_opts(eggsync_opts *o);

/*
 * eggsync_cluster -- EGG-SynC(D, eps) (Algorithm 4).
 *   points     : n*d float32, row-major, values in [0,1]; HOST memory
 *   n, d, eps  : sizes and the neighbourhood radius (L66)
 *   labels_out : n int32 (host); cluster id per point, clusters numbered
 *                0..k-1 by their smallest point index (canonical)
 *   iters_out  : number of Eq.1 updates applied (Alg 4's t at exit)
 * Returns EGGSYNC_OK, EGGSYNC_NOT_CONVERGED, or a negative error code.
 */
int eggsync_cluster(const float *points, int64_t n, int32_t d, float eps, int32_t *labels_out,
                    int32_t *iters_out);

/* As eggsync_cluster with options (device pointers, stream, stats, coords_out, max_iters).
 * Small inputs (n <= 4096, n*d <= 8192, d <= 8, the cell key in 64 bits, GRID mode, no
 * stats requested) run Algorithm 4 (L258-278) in ONE kernel launch -- a 16-CTA thread-block
 * cluster holding the state in distributed shared memory, no per-iteration host round trip
 * (SURVEY.md §8(f) F1); the same readings and results as the grid path (environment
 * EGGSYNC_SMALL=0 forces the grid path). */
int eggsync_cluster_ex(const float *points, int64_t n, int32_t d, float eps, const eggsync_opts *opts,
                       int32_t *labels_out, int32_t *iters_out);

/*
 * eggsync_step -- one pass of the loop body of Algorithm 4 on the caller's
 * state (for testing / resuming):
 *   points     : in D^t, out D^{t+1} (one synchronous Eq.1 update), n*d row-major float32, host
 *   synced_out : 1 iff the synchronization criterion (Def 4.2 in its grid
 *                form: first term |cell(p)| == |N_eps(p)| for all p, L252;
 *                second term L108-110, L254) holds on D^t, else 0
 */
int eggsync_step(float *points, int64_t n, int32_t d, float eps, int32_t *synced_out);

/*
 * As eggsync_step with options.  first_term_out / second_term_out may be NULL;
 * second_term_out is -1 when the first term fails (the paper only checks the
 * second term when the first holds, Alg 4 l.9-10 L273-275).
 */
int eggsync_step_ex(float *points, int64_t n, int32_t d, float eps, const eggsync_opts *opts,
                    int32_t *first_term_out, int32_t *second_term_out);

/* Thread-local message describing the last non-OK return of this thread. */
const char *eggsync_last_error(void);

/* Library version string. */
const char *eggsync_version(void);

/* The library keeps the most recently released device workspace of each
 * device (and its pinned flag buffer) cached for reuse by the next call that
 * fits in it, so repeated calls do not pay cudaMalloc/cudaFree.  This frees
 * the cache.  Not to be called concurrently with other library calls. */
void eggsync_release_cache(void);

/* ------------------------------------------------------------------------
 * Context (phase) API -- device-resident state for the multi-GPU driver and
 * for device-timed benchmarking.  Every pointer below is DEVICE memory on
 * the context's device; every call is asynchronous on the context's stream
 * except where a host output is written (then the call synchronises).
 *
 * Multi-GPU scheme: each rank holds all n points,
 * builds the identical grid (deterministic), updates only its contiguous
 * range [lo, hi) of the sorted order, and the caller all-gathers the owned
 * ranges (NCCL via torch.distributed) between eggsync_ctx_update and
 * eggsync_ctx_advance.  The termination flags are reduced with MIN.
 * ---------------------------------------------------------------------- */
typedef struct eggsync_ctx eggsync_ctx;

/* Create a context for n points of d dims; stream may be NULL (library-owned). */
int eggsync_ctx_create(int64_t n, int32_t d, float eps, int32_t device, void *stream, eggsync_ctx **out);
void eggsync_ctx_destroy(eggsync_ctx *ctx);

/* Load D^0: points is n*d row-major float32 (device pointer if on_device, else host). Validates [0,1]. */
int eggsync_ctx_load(eggsync_ctx *ctx, const float *points, int32_t on_device);

/* Build structure for the current state: cell keys, radix sort, cell offsets,
 * cell summaries, subtree hierarchy (L139-220 §4.2, Eq.5-6).
 * n_cells_out (host, may be NULL) receives the number of non-empty cells. */
int eggsync_ctx_build(eggsync_ctx *ctx, int32_t *n_cells_out);

/* EGG-update (Alg 3) of the sorted positions [lo, hi) into the next-state
 * buffer, plus the first-term flag of those points (device int32, AND-reduced). */
int eggsync_ctx_update(eggsync_ctx *ctx, int64_t lo, int64_t hi);

/* Second term of Def 4.2 (L108-110, L254) for sorted positions [lo, hi) on the current state. */
int eggsync_ctx_second_term(eggsync_ctx *ctx, int64_t lo, int64_t hi);

/* Read the flags: first = AND over updated points since the last build; second
 * = AND over checked points (-1 if never checked since the last build).  Synchronises. */
int eggsync_ctx_flags(eggsync_ctx *ctx, int32_t *first_out, int32_t *second_out);

/* Device pointers of the state: cur = D^t (SoA [d][n], sorted order), next = D^{t+1}
 * being written by eggsync_ctx_update. */
float *eggsync_ctx_cur_coords(eggsync_ctx *ctx);
float *eggsync_ctx_next_coords(eggsync_ctx *ctx);

/* Pack next-state columns [lo, lo+cnt) into buf (device, [d][cnt]); unpack a
 * gathered buffer ([ranks][d][cnt], rank r owning [r*cnt, min(n,(r+1)*cnt)))
 * into the next-state buffer.  Used around an NCCL all-gather. */
int eggsync_ctx_pack(eggsync_ctx *ctx, int64_t lo, int64_t cnt, float *buf);
int eggsync_ctx_unpack(eggsync_ctx *ctx, const float *gathered, int32_t ranks, int64_t cnt);

/* Make D^{t+1} the current state (t <- t+1). */
int eggsync_ctx_advance(eggsync_ctx *ctx);

/* Labels of the current state's cells (gatherCluster L256), canonical, written
 * to labels (n int32, device if on_device else host), original point order. */
int eggsync_ctx_labels(eggsync_ctx *ctx, int32_t *labels, int32_t on_device);

/* Current coordinates in original point order, n*d row-major (device if on_device). */
int eggsync_ctx_coords(eggsync_ctx *ctx, float *coords, int32_t on_device);

/* Run the whole loop (Alg 4) on the context's state; iters_out (host). */
int eggsync_ctx_run(eggsync_ctx *ctx, int32_t max_iters, int32_t *iters_out);

/* Stream of the context (cudaStream_t). */
void *eggsync_ctx_stream(eggsync_ctx *ctx);

/* Work counters of the update kernel (for the roofline).
 * enable = 1: reset the counters and run subsequent updates in the instrumented
 * variant; 0: back to the plain variant; -1: leave as is.  totals_out (host, 8
 * int64, may be NULL) receives, before the enable takes effect: [0] (point,cell)
 * classifications, [1] summary/point accumulations, [2] (point,point) scan tests,
 * [3] (point,subtree) box tests, [4] fp64 re-decisions, [5] (point,partial cell)
 * pairs, [6] full-subtree uses, [7] staged cells.  Synchronises. */
int eggsync_ctx_work(eggsync_ctx *ctx, int32_t enable, int64_t *totals_out);

/* Work and time of the tensor-core update kernel (the A6 path taken when d <= 12;
 * DESIGN.md §6), for its roofline.  enable = 1: reset and time every subsequent
 * tensor-core update launch with CUDA events on the context stream; 0: stop timing;
 * -1: leave as is.  out (host, 5 int64, may be NULL) receives the totals since the
 * last reset, before the enable takes effect: [0] tensor-core update launches,
 * [1] (point, entry) pairs (128 points x the tile's entries, padding excluded),
 * [2] pairs including the padding of the last entry tile, [3] algorithmic
 * tensor-core FLOPs 2*pairs*((3d+2) + 2(2d+1)), [4] summed kernel time in ns
 * (k_update_tc only; the plan pass is not included).  Synchronises on the last
 * timed launch.  Returns EGGSYNC_EINVAL for a NULL ctx. */
int eggsync_ctx_tc_work(eggsync_ctx *ctx, int32_t enable, int64_t *out);

/* Number of kernel launches this context has issued (CUB's internal launches
 * counted per pass). */
int64_t eggsync_ctx_launches(eggsync_ctx *ctx);

/* Block-interleaved ownership for load balance across ranks: the update works on
 * blocks of B = 64 (d <= 12) or 32 consecutive sorted points; rank r of `ranks`
 * owns the blocks b with b % ranks == r (dense and sparse regions are spread over
 * all ranks).  update_owned updates the owned points (like eggsync_ctx_update);
 * owned_count returns the per-rank exchange size cnt = ceil(nblocks/ranks)*B;
 * pack_owned writes the owned part of D^{t+1} to buf ([d][cnt], device, zero
 * padded); unpack_owned scatters a gathered [ranks][d][cnt] device buffer back. */
int eggsync_ctx_update_owned(eggsync_ctx *ctx, int32_t rank, int32_t ranks);
int64_t eggsync_ctx_owned_count(eggsync_ctx *ctx, int32_t ranks);
int eggsync_ctx_pack_owned(eggsync_ctx *ctx, int32_t rank, int32_t ranks, float *buf);
int eggsync_ctx_unpack_owned(eggsync_ctx *ctx, const float *gathered, int32_t ranks);

/* Sharded runs (distributed.run_sharded): the context holds a rank's own
 * points -- the first n_own of the loaded points -- followed by its halo (the other ranks'
 * points within eps+delta of the own ones).  Every point is updated, but only own points
 * contribute to the criterion flags (first term in the update, second term).  n_own >= n
 * (the default) means all points are own.  Errors: EINVAL. */
int eggsync_ctx_set_own(eggsync_ctx *ctx, int64_t n_own);

/* Collective choice of the update kernel (tensor-core or SIMT) for a multi-rank update, so
 * that every rank -- and one GPU running the whole range -- choose alike and the result stays
 * bitwise identical to one GPU.  eggsync_ctx_plan_owned runs the tensor-core plan pass
 * (Alg 3's neighbour-cell enumeration, L248) for the owned tiles only and writes six host
 * int64 statistics to stats_out: [0] entries, [1] points in entries, [2] owned tiles,
 * [3] plan overflow (0/1), [4] largest cell count, [5] tensor cores enabled (0/1).  The
 * caller reduces them over the ranks -- SUM of [0..2], MAX of [3..5] -- and passes the
 * result to eggsync_ctx_update_planned, which chooses from the global statistics and runs
 * the update of the owned tiles (reusing the plan).  Between the two calls nothing else may
 * run on the context.  Synchronous (the plan statistics are read back to the host).
 * Errors: EINVAL (bad rank / ranks, no build, NULL stats); ECUDA. */
int eggsync_ctx_plan_owned(eggsync_ctx *ctx, int32_t rank, int32_t ranks, int64_t *stats_out);
int eggsync_ctx_update_planned(eggsync_ctx *ctx, int32_t rank, int32_t ranks, const int64_t *global_stats);

/* ------------------------------------------------------------------------
 * Direct SynC (GPU-SynC-style) cross-check and the cluster order parameter
 * (SURVEY.md §8(f) F4).  No grid, no Eq.5 identity: every point is tested
 * against every point (O(n^2 d) per update), as the GPU-SynC baseline the
 * paper compares against does (L284: "distribute updates of all points among
 * threads").  A second, independent GPU path for Eq.1 and a speed floor for
 * the grid path; not used by eggsync_cluster.
 * ---------------------------------------------------------------------- */

/*
 * eggsync_sync_step -- one synchronous Eq.1 update (L68, Alg 1 l.3-5 L50-53)
 * computed directly, plus the cluster order parameter of the input state
 * (Eq.2, Alg 1 l.6 L54):
 *   r_c = 1/n * sum_p 1/|N_eps(p^t)| * sum_{q in N_eps(p^t)} exp(-||q^t - p^t||).
 *   points    : in D^t, out D^{t+1}; n*d float32 row-major; device memory when
 *               on_device = 1 (runs on the legacy default stream), else host.
 *               Coordinates are used as given (no [0,1] check: Eq.1 needs no grid).
 *   n, d, eps : 1 <= n <= 2^31-1, 1 <= d <= EGGSYNC_MAX_D, eps finite > 0.
 *   rc_out    : host double, r_c of D^t (may be NULL).
 *   nbr_out   : n int32, |N_eps(p^t)| (device when on_device, else host; may be NULL).
 * N_eps membership (||p-q|| <= eps, p in N_eps(p), L66) is decided exactly: fp32
 * distances outside a (4d+16)u relative band around eps^2 decide directly, the
 * rest are re-decided in fp64 as sum_i (q_i - p_i)^2 in dimension order.  Sums of
 * sin(q_i - p_i) (fp32 sinf) and exp(-||.||) (fp32) are accumulated per 128-point
 * tile in fp32 and in fp64 across tiles; the update and the mean are fp64 -> the
 * output float32.  Allocates O(n*d) device scratch per call.  Synchronises.
 * Returns EGGSYNC_OK, EGGSYNC_EINVAL, EGGSYNC_ENOMEM or EGGSYNC_ECUDA.
 */
int eggsync_sync_step(float *points, int64_t n, int32_t d, float eps, int32_t on_device, double *rc_out,
                      int32_t *nbr_out);

/*
 * eggsync_sync_lambda -- SynC with lambda-termination (Algorithm 1, L46-56),
 * GPU-SynC style: repeat { r_c = Eq.2 on D^t; D^{t+1} = Eq.1(D^t); t += 1 }
 * while r_c < lambda and t < max_iters (the update of the iteration whose r_c
 * reaches lambda is applied, as Alg 1 l.5-6 order it).  The paper's point
 * (Fig 1 L89, L95) is that this stops before the exact criterion holds; the
 * state returned in points can be handed to eggsync_step to see it.
 *   points, n, d, eps, on_device : as eggsync_sync_step.
 *   lambda    : threshold (Böhm et al. use 0.999, L77); max_iters >= 1.
 *   iters_out : updates applied (host, may be NULL); rc_out : last r_c (host, may be NULL).
 * Returns EGGSYNC_OK when r_c >= lambda was reached, EGGSYNC_NOT_CONVERGED at
 * max_iters, or a negative error code.
 */
int eggsync_sync_lambda(float *points, int64_t n, int32_t d, float eps, double lambda, int32_t max_iters,
                        int32_t on_device, int32_t *iters_out, double *rc_out);

#ifdef __cplusplus
}
#endif
#endif /* EGGSYNC_H */
