/*
 * mf.h -- C ABI of the B200-native multifrontal sparse SPD Cholesky hot path.
 *
 * The problem statement is the paper's [PAPER.md L7, Sec. I]: "For SPD linear
 * systems, the solution involves a Cholesky factorization of the coefficient
 * matrix A into LL^T, followed by a forward triangular solve Ly = b and a
 * backward triangular solve L^T x = y."  The factorization is the supernodal
 * multifrontal method of [PAPER.md L27, Sec. II-A]: a postorder traversal of the
 * supernodal elimination tree; per supernode n the frontal matrix F^n is built
 * from A's entries and the children's update matrices by extend-add, then the
 * factor-update (F-U) step -- potrf on L1^n (k x k), trsm on L2^n (m x k), and
 * U^n = U^n - L2^n L2^nT (syrk) [Fig. 1, PAPER.md L33-65] -- produces L and
 * the update matrix passed to the parent.
 *
 * Conventions:
 *   - Input matrix: 0-based CSC, n columns.  colptr: int64[n+1] (monotone,
 *     colptr[0] = 0); rowind: int32[colptr[n]] (need not be sorted).  Only
 *     entries with row >= col are read (LAPACK uplo='L'); upper entries are
 *     ignored, so a full symmetric CSC works too.  Duplicates are summed in
 *     input order.  A missing diagonal counts as 0 (=> not SPD).
 *   - perm: int32[n], perm[k] = original index of the k-th pivot (new -> old,
 *     as in A(p,p)).  The library composes it with an elimination-tree
 *     postorder; mf_get_perm() returns the composition ("final perm").
 *     perm == NULL: the library orders A itself on the host by METIS nested
 *     dissection (METIS_NodeND of the CUDA toolkit's static METIS, the ordering
 *     behind cusolverSpXcsrmetisndHost) of the graph of A + A^T; the paper used
 *     its solver's own ordering [PAPER.md L71].
 *   - values, b, x: float64 arrays that may be HOST or DEVICE pointers
 *     (detected with cudaPointerGetAttributes).  They are borrowed for the
 *     duration of the call only.  x is caller-allocated (n doubles) and must
 *     not alias b.  Device inputs must be complete when read: a ctx running on
 *     its own stream (mf_options.stream == NULL) first waits for the work
 *     already queued on the legacy default stream; a caller that passes its own
 *     stream orders the producers of values / b on that stream itself.
 *   - Ownership: the ctx owns the symbolic plan, the device arena (L panels
 *     and update matrices) and its CUDA stream usage until mf_destroy().
 *   - State machine: create -> analyze -> factor -> solve*; factor may repeat
 *     with new values of the same pattern; analyze resets.  Calls out of order
 *     return MF_ERR_STATE.
 *   - Errors: 0 = OK; negative = usage/resource errors (below); positive
 *     MF_NOT_SPD = a pivot was <= 0 or NaN: info.failed_col holds the ORIGINAL
 *     index of the first failing pivot in final-perm order, the factor is
 *     invalid and mf_solve returns MF_ERR_STATE.
 *   - Thread safety: one ctx per host thread; no global mutable state.
 */
#ifndef MF_H
#define MF_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MF_OK 0
#define MF_NOT_SPD 1
#define MF_ERR_ARG (-1)
#define MF_ERR_STATE (-2)
#define MF_ERR_NOMEM (-3)
#define MF_ERR_CUDA (-4)
#define MF_ERR_NCCL (-5)

typedef struct mf_ctx mf_ctx;

typedef struct {
    int32_t amalgamate;       /* 1 = SURVEY Appendix-B relaxed rule (default), 0 = fundamental supernodes */
    int32_t nrelax[3];        /* default {4, 16, 48}                                              */
    double zrelax[3];         /* default {0.8, 0.1, 0.05}                                         */
    int32_t small_front_max;  /* threshold policy (no variant model set): fronts of order <= this use
                                 the batched warp / shared-memory kernels, larger ones the tiled
                                 path; also the small/large split of the solve.  With a variant
                                 model (mf_set_variant_model) the model picks each front's class
                                 and this threshold does not bound it.                            */
    int32_t panel_w;          /* large-front diagonal block width (multiple of 16, <= 64)          */
    int32_t device;           /* CUDA device ordinal (-1 = current)                                */
    int32_t host_only;        /* 1 = symbolic analysis + planning only, no device (mf_factor/mf_solve
                                 then return MF_ERR_STATE); lets CPU-only hosts inspect the plan   */
    int32_t nranks;           /* GPUs (one process each) sharing the factorization (default 1)     */
    int32_t rank;             /* this process's rank in [0, nranks)                                 */
    void *stream;             /* cudaStream_t to run on (NULL = the ctx creates its own)           */
    int32_t split_all;        /* multi-GPU mapping: 0 (default) = choose the frontier and which top
                                 fronts are shared by the exchange-cost model; 1 = always split (a
                                 frontier of >= nranks subtrees, every eligible top front shared),
                                 e.g. to exercise the cooperative path on small problems           */
    int32_t nbranch;          /* single GPU: elimination subtrees are split into this many branches
                                 that run concurrently (CUDA-graph branches on their own streams)
                                 below the top fronts; 1 = one stream (default 4)                  */
    int32_t fuse_ea;          /* 1 (default) = the extend-add of the children's U^c into the U^s part
                                 of a large front is fused into the prologue of its syrk (the Schur
                                 update starts from the gathered sum 0 + U^c1 + U^c2 + ... instead of
                                 a U^s assembled in HBM); 0 = the
                                 assembly kernel builds the whole front.  Both give bit-identical
                                 fronts (same summation order, reading C6).                         */
    int32_t lookahead;        /* 1 = single GPU, main stream: each trailing update of a
                                 large front is split into the columns the next panel needs and the
                                 rest, which runs on a low-priority side stream beside that panel
                                 (the paper's overlap of CPU and GPU work [P:L325] as overlap of the
                                 latency-bound panel with throughput-bound updates); 0 (default) =
                                 one stream.  Same arithmetic either way (bit-identical L); measured
                                 no faster on c3-c5 (the co-running update slows the panel chain). */
    /* Device-memory hooks (NULL = cudaMalloc / cudaFree).  Every device buffer the
     * ctx owns (plan arrays, L and U arenas, vectors) is taken from dev_alloc(bytes,
     * alloc_user) on the ctx's device and returned through dev_free(ptr, alloc_user)
     * by mf_analyze (re-analysis) and mf_destroy; the Python binding can route them
     * to PyTorch's caching allocator.  dev_alloc returns NULL on failure
     * (=> MF_ERR_NOMEM).  Both or neither must be set. */
    void *(*dev_alloc)(size_t bytes, void *alloc_user);
    void (*dev_free)(void *ptr, void *alloc_user);
    void *alloc_user;
    /* Schur updates (the SYRK/GEMM of every large front) on the int8 tensor cores
     * (tcgen05.mma .kind::i8, TMEM accumulators) by the Ozaki scheme: each row of
     * the panel is scaled by a power of two and cut into ozaki_slices signed 7-bit
     * digits; digit products are exact in int32 and recombined in fp64 (SURVEY.md
     * NEXT-3; Sec. III-B: the paper's GPU part ran in single
     * precision with double-precision refinement).
     *   0 (default) = FP64 DMMA (mma.sync.m8n8k4.f64);
     *   8 = FP64-class emulation (digit truncation 2^-56 of the row scales);
     *   3..7 = reduced precision; mf_solve then refines in fp64 (refine_iters).
     * Update launches with a short average inner dimension (< 2048, where DMMA
     * measured faster) stay on DMMA.  Forces lookahead = 0. */
    int32_t ozaki_slices;
    /* mf_solve: maximum fp64 iterative-refinement steps x += A^{-1}(b - A x) with
     * the residual in fp64 from the original values; stops when the backward error
     * ||b - A x||_inf / (||A||_inf ||x||_inf + ||b||_inf) <= 2^-52 or stops
     * decreasing.  -1 (default) = auto: 0 for ozaki_slices 0 or 8, else 10. */
    int32_t refine_iters;
} mf_options;

typedef struct {
    int64_t n;
    int64_t nnzA;             /* entries read (row >= col) */
    int64_t nnzL;             /* true nnz(L) = sum of column counts */
    int64_t nnzL_stored;      /* sum over supernodes of k(k+1)/2 + k m */
    int64_t panel_words;      /* sum over supernodes of ldL * k (device storage of L) */
    int64_t flops_true;       /* sum cc_j^2 (SURVEY Sec. 8(a) flop accounting) */
    int64_t flops_exec;       /* sum over fronts of k m^2 + m k(k+1) + k(k+1)(2k+1)/6 */
    int32_t nfund;            /* fundamental supernodes */
    int32_t nsuper;           /* supernodes after amalgamation */
    int32_t nlevels;          /* levels of the bottom-up schedule */
    int32_t max_front;        /* largest f = k + m */
    int64_t rows_total;       /* sum over supernodes of f (length of the row lists) */
    int64_t failed_col;       /* original index of the first failing pivot, or -1 */
    int64_t workspace_bytes;  /* device bytes held by the ctx */
    int64_t launches_factor;  /* kernel launches issued by one mf_factor */
    double t_analyze;         /* seconds (host wall) of the last mf_analyze */
    double t_factor;          /* seconds (device events) of the last mf_factor */
    double t_solve;           /* seconds (device events) of the last mf_solve */
    int32_t nbranch;          /* concurrent subtree branches the factorization uses (single GPU)   */
    int32_t ozaki_slices;     /* Schur-update mode in use (mf_options.ozaki_slices)                 */
    int32_t refine_steps;     /* refinement steps taken by the last mf_solve                        */
    double solve_berr;        /* backward error of the last mf_solve's x when refinement ran, else -1 */
    int64_t launches_ozaki;   /* Schur-update launches of mf_factor on the int8 tensor cores       */
} mf_info;

/* Per-kernel-class statistics of profiled factorizations (mf_set_profiling):
 * CUDA-event time on the ctx stream around every launch of the class, and the
 * ALGORITHMIC flops / HBM bytes of those launches. */
typedef struct {
    char name[32];
    int64_t launches;
    double ms;
    double flops;
    double bytes;
} mf_kernel_stat;

#define MF_KERNEL_CLASSES 7

/* Multi-GPU exchange.  With nranks > 1 every rank makes the
 * same calls with the same n/colptr/rowind/perm; `values` and `b` are read from
 * RANK 0's buffers and broadcast (other ranks may pass any buffer of the right
 * size); x is returned on every rank.  Elimination subtrees are mapped to ranks;
 * the supernodes above them ("top") are replicated on every rank, the small ones
 * factored redundantly and the large ones cooperatively (pivot-column blocks
 * owned block-cyclically and broadcast by their owner, U^n all-gathered;
 * DESIGN.md Sec. 9).  The library hands
 * the data movement to a caller-supplied callback (NCCL through torch.distributed
 * in the Python binding), called by every rank with matching lists:
 *   SEND/RECV  point-to-point, `peer` = the other rank;
 *   BCAST      in place, root = `peer`;
 *   ALLREDUCE_SUM (float64) / ALLREDUCE_MIN_I32 (int32), in place.
 * Buffers are device pointers; the ctx stream is synchronized before the call and
 * the callback must return only when the transfers are complete (0 = success). */
#define MF_XFER_SEND 1
#define MF_XFER_RECV 2
#define MF_XFER_BCAST 3
#define MF_XFER_ALLREDUCE_SUM 4
#define MF_XFER_ALLREDUCE_MIN_I32 5
typedef struct {
    int32_t op;
    int32_t peer;
    void *ptr;
    int64_t bytes;
} mf_xfer;
typedef int (*mf_exchange_fn)(void *user, const mf_xfer *ops, int64_t nops);

/* Fill *opt with the defaults. */
int mf_default_options(mf_options *opt);

/* Create a context.  opt may be NULL (defaults). */
int mf_create(mf_ctx **ctx, const mf_options *opt);

/* Symbolic analysis + device planning for the pattern (colptr, rowind) under
 * the order perm; perm == NULL = METIS nested
 * dissection computed here (see "perm" above).  Host arrays only.  Uploads the
 * flat plan arrays and allocates the device arena.  Errors: MF_ERR_ARG for a
 * malformed pattern or a perm that is not a permutation. */
int mf_analyze(mf_ctx *ctx, int64_t n, const int64_t *colptr, const int32_t *rowind,
               const int32_t *perm);

/* Numeric factorization A = L L^T (rows a1-a8): values[colptr[n]] aligned with
 * rowind, host or device.  Runs on the ctx stream and synchronizes it before
 * returning (the NOT_SPD flag is read back). */
int mf_factor(mf_ctx *ctx, const double *values);

/* x = A^{-1} b through L y = P b, L^T z = y, x = P^T z [PAPER.md L7].
 * b, x host or device (n doubles each, not aliased). */
int mf_solve(mf_ctx *ctx, const double *b, double *x);

/* nrhs right-hand sides: B and X are column-major n x nrhs with leading
 * dimensions ldb, ldx >= n (host or device, not aliased); X(:, r) = A^{-1} B(:, r),
 * bitwise the same as nrhs calls of mf_solve.  Single GPU: up to 8 solve
 * pipelines (own vectors, flags, streams and CUDA graphs, allocated on first use)
 * run right-hand sides concurrently, overlapping the latency-bound block chains of
 * the large supernodes; one final synchronization.  With several ranks or with
 * refinement: one mf_solve per column.  MF_ERR_ARG for nrhs < 0 or ld < n. */
int mf_solve_nrhs(mf_ctx *ctx, int32_t nrhs, const double *B, int64_t ldb, double *X, int64_t ldx);

int mf_get_info(const mf_ctx *ctx, mf_info *out);

/* final_perm[n]: perm composed with the postorder (new -> old). */
int mf_get_perm(const mf_ctx *ctx, int32_t *final_perm);

/* Elimination tree (final labels) and column counts: parent[n] (-1 = root),
 * colcount[n] (incl. diagonal).  Host buffers. */
int mf_get_etree(const mf_ctx *ctx, int32_t *parent, int64_t *colcount);

/* Supernode partition after amalgamation (host buffers):
 * sn_first[nsuper+1], sn_parent[nsuper], sn_rowptr[nsuper+1],
 * sn_rows[rows_total] (R_s ascending, first k entries = the pivot columns).
 * fund_first[nfund+1] = fundamental partition (may be NULL). */
int mf_get_supernodes(const mf_ctx *ctx, int32_t *sn_first, int32_t *sn_parent, int64_t *sn_rowptr,
                      int32_t *sn_rows, int32_t *fund_first);

/* Copy the L panel of supernode s to host memory: out[f * k], column-major
 * with leading dimension f (rows R_s, columns cols(s)); the strict upper
 * triangle of the k x k block is zero.  Requires a successful mf_factor. */
int mf_export_panel(const mf_ctx *ctx, int32_t s, double *out);

/* Diagonal of L in final-perm order: out[n] (host).  log det A = 2 sum log out[j]. */
int mf_export_diag(const mf_ctx *ctx, double *out);

/* Copy every panel (supernode order, each f*k as above) to host: out[sum f*k]. */
int mf_export_panels(const mf_ctx *ctx, double *out);

/* L in supernodal CSC (final-perm labels, host buffers): column j of supernode s
 * (local column jj) holds the rows R_s[jj..f) -- its diagonal first, then the
 * rows below, ascending -- so Lp[n] = info.nnzL_stored; entries that are
 * amalgamation padding are stored as exact 0.0.  Lp: int64[n + 1],
 * Li: int32[nnzL_stored], Lx: float64[nnzL_stored]; any of them may be NULL
 * (e.g. Lp alone to size the others).  Requires a successful mf_factor (Lp / Li
 * alone: a successful mf_analyze). */
int mf_export_L(const mf_ctx *ctx, int64_t *Lp, int32_t *Li, double *Lx);

/* The static launch program mf_factor replays (one entry per kernel launch, in
 * order; the leading init launch is not listed).  kind = kernel class index
 * (order of mf_kernel_stat), count = CTAs (tasks) of the launch. */
typedef struct {
    int32_t kind;
    int32_t level;
    int64_t count;
    double flops;
    double bytes;
    double int8_ops;   /* Schur update on the int8 tensor cores (ozaki_slices): int8 MMA
                          operations executed (2 x MACs, padding included), else 0 */
    int32_t stream;    /* single GPU: subtree branch (CUDA-graph branch) of the launch, -1 = main */
    int32_t reserved;
} mf_launch_info;

/* out may be NULL to query *count only. */
int mf_get_program(const mf_ctx *ctx, mf_launch_info *out, int64_t max, int64_t *count);

/* Register the exchange callback (required before mf_factor when nranks > 1). */
int mf_set_exchange(mf_ctx *ctx, mf_exchange_fn fn, void *user);

/* Subtree-to-GPU mapping of the analyzed pattern: owner[nsuper] (rank factoring
 * each supernode) and top[nsuper] (0 = in a rank's subtree; 1 = top supernode,
 * replicated and factored redundantly by every rank; 2 = top supernode factored
 * cooperatively: pivot-column blocks block-cyclic over the ranks, broadcast by
 * their owner, U^n all-gathered).
 * rank_load[nranks] = executed flops of each rank's subtrees; *top_load = flops
 * of the top.  Any pointer may be NULL. */
int mf_get_mapping(const mf_ctx *ctx, int32_t *owner, int8_t *top, double *rank_load, double *top_load);

/* Per-launch CUDA-event timing in mf_factor; resets the stats.  enable = 1: the
 * launches run eagerly on one stream, an event around each (serialised: per-kernel
 * times); 2: timeline -- the factorization runs as its usual CUDA graph (subtree
 * branches and streams concurrent), with timing events captured before and after
 * every launch (mf_get_launch_timeline); 0: off. */
int mf_set_profiling(mf_ctx *ctx, int enable);

/* out[MF_KERNEL_CLASSES]: accumulated stats since the last mf_set_profiling; *count = classes written. */
int mf_get_kernel_stats(const mf_ctx *ctx, mf_kernel_stat *out, int32_t *count);

/* Per-launch CUDA-event times (ms) of the last PROFILED factorization, in program
 * order (mf_get_program; the local program only).  out may be NULL to query *count. */
int mf_get_launch_times(const mf_ctx *ctx, double *out_ms, int64_t max, int64_t *count);

/* Timeline of the last factorization run with mf_set_profiling(ctx, 2): for every
 * launch of the local program (program order, mf_get_program) the times (ms) at
 * which its stream reached it and finished it, relative to the start of the
 * factorization, as the concurrent graph ran -- the critical path of the
 * schedule, not per-kernel costs.  start_ms / end_ms may be NULL (both NULL:
 * *count only).  MF_ERR_STATE unless such a factorization ran.  Multi-GPU: the
 * local program only. */
int mf_get_launch_timeline(const mf_ctx *ctx, double *start_ms, double *end_ms, int64_t max, int64_t *count);

/* Learned kernel-variant selector (Sec. VI, Eqs. 3-5).
 * The paper picks a CPU/GPU policy per factor-update call with a cost-sensitive
 * multinomial logistic classifier y(x) = argmax_j x . theta_j over front features
 * x(m, k).  Here the classes are GPU kernel variants of a front:
 *   0: one warp per front, f <= 16        1: one warp per front, f <= 32
 *   2: one CTA per front in shared memory, f <= 64     3: ... f <= 96
 *   4: ... f <= 128      5: ... f <= 160      6: tiled large-front path (any f)
 * and x = [1, m/64, k/64, m/k, (m/64)^2, (m/64)(k/64), (k/64)^2, (k/64)^3, (m/64)(k/64)^2]
 * (the paper's [m, k, m/k, m^2, mk, k^2, k^3, mk^2] after a constant, m and k in
 * units of 64).  theta: MF_VARIANT_FEATURES x MF_VARIANTS row-major (theta[q * MF_VARIANTS
 * + j] = weight of feature q for class j); NULL = the default front-order thresholds.
 * force >= 0 forces class `force` wherever it is feasible (used to measure the
 * per-class times the model is fitted to).  Call before mf_analyze; the choice is
 * made once per pattern.  Returns MF_ERR_STATE after mf_analyze, MF_ERR_ARG for a
 * bad class or size. */
#define MF_VARIANTS 7
#define MF_VARIANT_FEATURES 9
int mf_set_variant_model(mf_ctx *ctx, const double *theta, int32_t nfeatures, int32_t nclasses, int32_t force);

/* Kernel-variant class of every supernode of the analyzed pattern: out[nsuper]. */
int mf_get_variants(const mf_ctx *ctx, int32_t *out);

void mf_destroy(mf_ctx *ctx);

const char *mf_strerror(int code);

#ifdef __cplusplus
}
#endif
#endif /* MF_H */
