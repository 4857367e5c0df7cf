/*
 * lu_sym.h — C ABI of the B200-native symbolic LU hot path.
 *
 * Implements, for a square sparse pattern A (CSR), the method of Xia et al., "End-to-End LU
 * Factorization of Large Matrices on GPUs" (PPoPP'23), /root/reference/PAPER.md:
 *
 *   S1  validate A                                            (input of Alg. 1; CSR L270)
 *   S3  lu_sym_count : per-row fill2 traversal, counts only   (symbolic_1, Alg. 3;
 *                                                               Alg. 1; Thm 1)
 *   S4  lu_sym_scan  : exclusive prefix sum of the counts     (prefix_sum, Alg. 3)
 *   S5  (caller)     : allocate col_idx_lu[nnz]                (Alg. 3)
 *   S6  lu_sym_emit  : the same traversal, writing positions  (symbolic_2, Alg. 3)
 *   S8/S9 lu_levelize: dependency graph, in-degrees, Kahn      (Alg. 5, level formula
 *                      topological levels                       L283, dependency rule L167)
 *
 * Conventions (all functions):
 *   - extern "C", no C++ or framework types.  Pointers named d_* are DEVICE pointers on the
 *     caller's current CUDA device; h_* / plain out-params are HOST pointers.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Work is
 *     stream-ordered on it; calls that return a host value (nnz, num_levels, status of input
 *     validation) synchronise that stream before returning.
 *   - Indices are 0-based (reading R1).  A's rows must be strictly increasing (sorted, no
 *     duplicates; reading R8).  The diagonal of L+U is present iff A(i,i) is (R7).
 *   - Output rows are sorted ascending (R9); fill_count[i] = |row i of L+U| including original
 *     entries and the diagonal (R10); offsets are int64 (R11).
 *   - Errors are returned as lu_status, never by abort/exception; lu_last_error() gives a
 *     thread-local message for the last failing call on this thread.
 *   - Ownership: A's arrays are BORROWED by the handle and must stay valid and unchanged until
 *     lu_sym_destroy.  Output arrays are CALLER-allocated.  The handle owns only its scratch.
 *   - Threading: one handle is used by one host thread at a time; distinct handles are
 *     independent.
 */
#ifndef LU_SYM_H
#define LU_SYM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LU_SYM_ABI_VERSION 2

typedef enum {
    LU_OK = 0,
    LU_ERR_ARG = 1,      /* null pointer, negative size, bad enum, row range out of [0,n]     */
    LU_ERR_INPUT = 2,    /* A is not a valid CSR pattern (see lu_sym_create)                 */
    LU_ERR_NOMEM = 3,    /* scratch budget smaller than one row's minimum scratch, or OOM   */
    LU_ERR_CAPACITY = 4, /* caller's output buffer smaller than nnz(L+U)                     */
    LU_ERR_CUDA = 5,     /* a CUDA runtime error (message in lu_last_error)                  */
    LU_ERR_STATE = 7,    /* wrong call order (e.g. emit before scan), or device-side check   */
    LU_ERR_INTERNAL = 8  /* a device-side consistency check failed (count/emit mismatch)     */
} lu_status;

/* Dependency rule for levelization (reading R12).
 *   LU_DEP_U    : column j depends on column i iff i<j and (i,j) in L+U
 *   LU_DEP_GLU3 : additionally iff i<j and (j,i) in L+U (our reading of the "other
 *                 dependencies" deferred to GLU3.0 at L167/L497; multi-edges counted once per
 *                 source entry, identically in in-degree and update). */
enum { LU_DEP_U = 0, LU_DEP_GLU3 = 1 };

/* lu_sym_opts.flags — tuning / test knobs (never change results) */
enum {
    LU_F_GLOBAL_BITMAP = 1 << 0, /* keep visited bitmaps in HBM slots even if smem would fit */
    LU_F_NO_BATCH = 1 << 1,      /* one threshold at a time, exactly Alg. 1's order (L130)   */
    LU_F_ASCENDING = 1 << 2,     /* process rows in increasing id (default: decreasing,
                                    i.e. heaviest-first)                      */
    LU_F_NO_PRUNE = 1 << 3,      /* levelize over every U edge (no transitive pruning)       */
    LU_F_KAHN_WIDE_ONLY = 1 << 4,/* levelize: never use the single-CTA narrow phase          */
    LU_F_NO_CONTRACT = 1 << 5,   /* levelize: Kahn over every column (no chain contraction)  */
    LU_F_TWO_PASS = 1 << 6,      /* no staging pool: emit re-runs the traversal (Alg. 3 as
                                    printed, symbolic_2 repeats symbolic_1's work)           */
    LU_F_ONE_CLASS = 1 << 7,     /* one row class (Alg. 3's single chunk size) instead of
                                    Alg. 4's row classes by scratch need (L272-277)          */
    LU_F_FORCE_CLASSES = 1 << 8, /* test knob: split row classes down to 64 shared words even
                                    when that does not add rows in flight                     */
    LU_F_SELF_CONT = 1 << 9,     /* BFS self-continuation (a lane expands its own first new
                                    vertex in the next round; the order below a threshold is
                                    free, reading R5) in every row class, not only in classes
                                    with one row per SM                                       */
    LU_F_NO_SELF_CONT = 1 << 10, /* no self-continuation anywhere (plain level-synchronous
                                    BFS)                                                      */
    LU_F_PAPER_CHUNKS = 1 << 11, /* Alg. 3's launch scheme (L239-243, L253-267): each pass is
                                    num_iter = ceil(rows / chunk_size) launches issued one
                                    after another, chunk_size = L / (c n) rows with c = 6
                                    4-byte words per vertex and L = the scratch budget (reading
                                    R16), chunks in increasing row order; with LU_F_ONE_CLASS
                                    this is Alg. 3, without it Alg. 4 (one chunk size per row
                                    class).  Ablation of the persistent heaviest-first launch
                                                                                */
    LU_F_MANAGED = 1 << 12,      /* unified-memory variant (Figs 5-6,
                                    Table 3): the traversal scratch (visited /
                                    done maps, frontier spill, L staging, staging pool, row
                                    offsets) comes from cudaMallocManaged and migrates to the
                                    GPU on first touch (page faults)                         */
    LU_F_MANAGED_PREFETCH = 1 << 13,/* with LU_F_MANAGED: cudaMemAdvise(preferred location =
                                    this GPU) + cudaMemPrefetchAsync after each allocation    */
    LU_F_NO_DEFER = 1 << 14,     /* no deferred rows: every row is finished by its fill2
                                    traversal (see lu_sym_opts.defer_windows)                 */
    LU_F_NO_SPARSE = 1 << 15,    /* planner: never replace shared-memory row classes by the
                                    sparse class (HBM visited slots, 16 rows per SM) that a
                                    create-time sample of rows selects when they visit < n/16
                                    vertices on average (reading G9)              */
    LU_F_COUNT_TE = 1 << 17,     /* a statistics handle: lu_sym_count counts the traversed
                                    edges of every scanned vertex, so stats.edges_read_count
                                    is the method's exact TE (reading R24); its count pass
                                    does not stage rows (lu_sym_emit then traverses again)   */
    LU_F_ASYNC_BFS = 1 << 18,    /* below-threshold traversal without level barriers (warp
                                    rings + a CTA pool; the order below a threshold is free,
                                    reading R5) in every row class of the 1024-thread
                                    one-CTA-per-SM kernel, not only in classes with at most
                                    2 rows per SM                                             */
    LU_F_NO_ASYNC_BFS = 1 << 19, /* level-synchronous BFS in every row class                 */
    LU_F_DEFER_GLOBAL = 1 << 16  /* row sharding (reading G8 across GPUs): lu_sym_count may
                                    defer rows even when the rows below them are counted on
                                    other GPUs; it then runs no tail: the deferred rows keep
                                    fill_count 0, lu_sym_deferred_flags reports them, and
                                    lu_sym_merge_deferred finishes them once the pattern of
                                    the other rows is assembled                              */
};

typedef struct {
    int32_t struct_size;           /* = sizeof(lu_sym_opts)                                  */
    int32_t flags;                 /* LU_F_*                                                 */
    uint64_t scratch_budget_bytes; /* 0 => 0.85 x free HBM at create (out-of-core planner)   */
    int32_t threads_per_row;       /* CTA size per row in flight; 0 => planner (128..1024);
                                      1025 = 1024 threads with the one-CTA-per-SM register
                                      budget (the planner picks it when shared memory allows
                                      only one 1024-thread CTA per SM anyway)               */
    int32_t rows_in_flight;        /* 0 => planner (all resident CTAs); > 0 caps it          */
    int32_t queue_capacity;        /* shared-memory frontier entries per buffer; 0 => planner */
    int32_t ell_width;             /* traversal adjacency slots 4, 6 or 8; 0 => planner     */
    uint64_t pool_bytes;           /* HBM staging pool for the rows found by lu_sym_count, so
                                      lu_sym_emit places them instead of re-traversing;
                                      0 => min(32 GiB, what the budget leaves)              */
    int32_t defer_windows;         /* deferred rows (reading G8): a row whose fill2
                                      threshold loop exceeds this many threshold windows is
                                      abandoned and finished after the pass by the row-merge
                                      closure over the rows below it, read from the staging
                                      pool (Theorem 1, split at the largest intermediate
                                      vertex).  Only rows whose lower rows are all staged by
                                      this handle qualify.  0 => 4096; < 0 => never          */
    int32_t defer_max;             /* at most this many deferred rows per call (0 => 1024,
                                      capped at 4096)                                       */
    int32_t reserved[4];
} lu_sym_opts;

typedef struct {
    double ms_create;             /* validate + adjacency build + planning                  */
    double ms_count, ms_scan, ms_emit, ms_levelize; /* last call of each (device events)     */
    int64_t nnz_lu;               /* after lu_sym_scan                                       */
    int64_t edges_read_count;     /* traversed edges (R24) of the last count / emit pass:    */
    int64_t edges_read_emit;      /*   exact with LU_F_COUNT_TE; without it only the entries
                                     read from A's CSR (seed rows, heavy rows)               */
    int64_t vertices_scanned_count, vertices_scanned_emit; /* scanned vertices (every
                                     threshold once + every BFS vertex), exact; rows deferred
                                     to the tail (G8) contribute what they scanned before    */
    int64_t spills;               /* frontier entries that spilled from smem to HBM          */
    int64_t scratch_bytes;        /* HBM scratch owned by the handle                         */
    int32_t rows_in_flight;       /* CTAs (= rows processed concurrently)                    */
    int32_t threads_per_row;
    int32_t smem_bytes_per_row;
    int32_t visited_in_smem;      /* top row class: 1 visited bitmap in shared memory, 0 in
                                     HBM slots, 2 split (part in shared memory, part in HBM) */
    int32_t ell_width;
    int32_t queue_capacity;
    int32_t num_levels;           /* after lu_levelize with this handle                      */
    int32_t levelize_wide_levels, levelize_narrow_levels; /* Kahn rounds by mode            */
    int32_t levelize_rank_rounds; /* pointer-jumping rounds of the chain contraction        */
    int32_t row_classes;          /* Alg. 4 row classes planned (1 = a single class)         */
    int32_t reserved[1];
    int64_t pool_bytes;           /* staging pool size (0: two-pass mode)                    */
    int64_t rows_retraversed;     /* rows of the last emit that were not staged              */
    int64_t kernel_launches;      /* kernels this handle launched since create (all calls)  */
    int64_t rows_deferred;        /* last count call: rows handed to the row-merge tail      */
    int64_t rows_merge_failed;    /* ... of which the tail could not finish (re-traversed)   */
    int64_t merge_entries_read;   /* ... strict-U entries of staged rows the tail read       */
    double ms_tail;               /* ... device time of the tail (included in ms_count)     */
    int64_t merge_rounds;         /* ... frontier rounds of the tail, summed over its rows   */
    int64_t merge_waits;          /* ... members that were deferred rows still in progress   */
    double sample_mean_sv;        /* planner: mean vertices scanned per sampled row (reading
                                     G9); -1 if create did not sample                        */
    int64_t heavy_rows;           /* rows of off-diagonal degree > ell_width, scanned by a
                                     whole warp from A's CSR instead of one ELL load         */
} lu_sym_stats;

typedef struct lu_sym lu_sym;

/* Library ABI version (== LU_SYM_ABI_VERSION). */
int32_t lu_sym_abi_version(void);

/* Fill *opts with defaults (struct_size set, everything else 0). */
void lu_sym_default_opts(lu_sym_opts *opts);

/*
 * Create a handle for the n x n pattern A given in CSR on the device:
 *   d_row_ptr : int64[n+1], d_row_ptr[0] = 0, non-decreasing, d_row_ptr[n] = nnz_a
 *   d_col_idx : int32[nnz_a], each row strictly increasing, values in [0, n)
 * Validates A on the device (LU_ERR_INPUT with the first offending row in lu_last_error),
 * builds the traversal adjacency and plans rows-in-flight from the scratch budget
 * (chunk_size = L/(c n); here slots = budget / per-row scratch).
 * n = 0 is allowed (every later call is a no-op).
 */
lu_status lu_sym_create(lu_sym **out, int32_t n, int64_t nnz_a, const int64_t *d_row_ptr,
                        const int32_t *d_col_idx, const lu_sym_opts *opts, void *stream);

/*
 * S3 — symbolic_1: for every row i in [row_begin, row_end) write
 *   d_fill_count[i] = |{ j : (i,j) in L+U }|      (int32[n] array indexed by global row id)
 * Entries outside the range are not touched (row sharding across GPUs).
 */
lu_status lu_sym_count(lu_sym *h, int32_t row_begin, int32_t row_end, int32_t *d_fill_count,
                       void *stream);

/*
 * S4 — exclusive prefix sum: d_row_ptr_lu[0] = 0, d_row_ptr_lu[i+1] = d_row_ptr_lu[i] +
 * d_fill_count[i] for all i < n (int64).  *nnz_lu (host) = d_row_ptr_lu[n].  Synchronises.
 */
lu_status lu_sym_scan(lu_sym *h, const int32_t *d_fill_count, int64_t *d_row_ptr_lu,
                      int64_t *nnz_lu, void *stream);

/*
 * S6 — symbolic_2: for every row i in [row_begin, row_end) write the sorted column ids of row i
 * of L+U to d_col_idx_lu[d_row_ptr_lu[i] .. d_row_ptr_lu[i+1]).  cap = number of int32
 * elements of d_col_idx_lu; LU_ERR_CAPACITY if cap < d_row_ptr_lu[row_end] (checked against
 * the handle's last scan).  LU_ERR_STATE if lu_sym_scan has not run on this handle.
 * LU_ERR_INTERNAL if a row's emitted length differs from its count (device check).
 */
lu_status lu_sym_emit(lu_sym *h, int32_t row_begin, int32_t row_end, const int64_t *d_row_ptr_lu,
                      int32_t *d_col_idx_lu, int64_t cap, void *stream);

/*
 * Convenience two-call protocol over all rows:
 *   call 1 with d_col_idx_lu == NULL: count + scan; sets *nnz_lu; returns LU_OK.
 *   call 2 with cap >= *nnz_lu: emit only (counts cached in the handle's scan).
 *   cap < nnz: LU_ERR_CAPACITY with *nnz_lu set; the handle stays usable.
 */
lu_status lu_sym_run(lu_sym *h, int32_t *d_fill_count, int64_t *d_row_ptr_lu,
                     int32_t *d_col_idx_lu, int64_t cap, int64_t *nnz_lu, void *stream);

/*
 * A-priori capacity of the pattern from A alone (no traversal): *bound (host) >= nnz(L+U).
 * By Theorem 1 ((i,j) fills iff a path i -> j has every intermediate vertex
 * < min(i,j)), row i of L+U lies in [min(i, min A(i,:)), max(i, max over u <= i of
 * max A(u,:))], and *bound is the sum of those row spans.  It is exact when every such span
 * fills (banded matrices, e.g. natural-ordered grids) and loose when a late dense row or
 * column widens the envelope (hub rows ordered last).  Lets a caller allocate the device and
 * host outputs before lu_sym_run_host instead of after a count pass.  Synchronises.
 */
lu_status lu_sym_nnz_bound(lu_sym *h, int64_t *bound, void *stream);

/*
 * Whole symbolic pass with the result streamed to the host while later rows are still being
 * traversed: Alg. 3's out-of-core chunks (L239-270) taken in INCREASING row order, nchunks row
 * ranges of equal a-priori traversal cost (0 => min(16, max(1, n/4096)); at most 64).  Per chunk: symbolic_1 with
 * staging (the traversal; chunk k+1 runs on a second scratch set so it fills the SMs chunk k
 * drains), the chained prefix sum of its counts (L262), symbolic_2 as a placement of its
 * staged rows (L264-270) and the device->host copy of its rows, the last three behind the
 * next chunks' traversal.
 *   d_fill_count [n], d_row_ptr_lu [n+1], d_col_idx_lu [cap]: device outputs, as lu_sym_run.
 *   h_row_ptr_lu [n+1], h_col_idx_lu [cap]: host copies (pinned memory overlaps the copies
 *   with the traversal; pageable works but serialises); either may be NULL.
 *   *nnz_lu (host) = nnz(L+U).  cap must be an upper bound of nnz(L+U) given up front;
 *   cap < nnz: LU_ERR_CAPACITY with *nnz_lu, d_fill_count and d_row_ptr_lu valid.
 * Blocks until the host copies are complete.  The handle is left scanned (lu_sym_emit and
 * lu_levelize may follow).  With LU_F_TWO_PASS (no staging pool) it runs lu_sym_run's two
 * calls and copies afterwards.  Allocates a second traversal scratch set on first use.
 */
lu_status lu_sym_run_host(lu_sym *h, int32_t nchunks, int32_t *d_fill_count,
                          int64_t *d_row_ptr_lu, int32_t *d_col_idx_lu, int64_t cap,
                          int64_t *h_row_ptr_lu, int32_t *h_col_idx_lu, int64_t *nnz_lu,
                          void *stream);

/*
 * S8+S9 — levelization (Algorithm 5) of the column-dependency DAG of the pattern
 * (d_row_ptr_lu int64[n+1], d_col_idx_lu int32[nnz], rows sorted as lu_sym_emit writes them):
 *   d_level[j] = 0 if column j has no predecessor, else 1 + max level of its predecessors
 *   (PAPER.md L283); *num_levels (host) = max level + 1 (0 if n = 0).  Synchronises.
 * dep_rule: LU_DEP_U or LU_DEP_GLU3.  h may be NULL (scratch allocated per call) or a handle
 * (scratch cached; stats recorded; its opts.flags LU_F_NO_PRUNE / LU_F_KAHN_WIDE_ONLY apply).
 */
lu_status lu_levelize(lu_sym *h, int32_t n, const int64_t *d_row_ptr_lu,
                      const int32_t *d_col_idx_lu, int32_t dep_rule, int32_t *d_level,
                      int32_t *num_levels, void *stream);

/*
 * Level-grouped column schedule (the form of Fig. 1(d), L72-80, consumed level by level by the
 * numeric phase, L206-208): from d_level[n] (levels in [0, num_levels), e.g. lu_levelize's
 * output) write d_level_ptr[num_levels+1] (int64) and d_level_cols[n] (int32) such that the
 * columns of level l are d_level_cols[d_level_ptr[l] .. d_level_ptr[l+1]), ascending (R15).
 * Synchronises.  LU_ERR_ARG on null pointers or num_levels < 1 with n > 0.
 */
lu_status lu_level_schedule(int32_t n, const int32_t *d_level, int32_t num_levels,
                            int64_t *d_level_ptr, int32_t *d_level_cols, void *stream);

/*
 * GLU3.0 level types, the per-level kernel-mode choice of the
 * numeric phase.  For level l (levels from lu_levelize): width = number of its columns,
 * d_sub[l] = total sub-columns of its columns, where the sub-columns of column j are the
 * columns k > j with (j,k) in L+U — the columns Alg. 2 (lines 7-14, L165-204) updates from
 * column j, i.e. its out-edges under LU_DEP_U (reading R28).  d_type[l] =
 *   LU_LEVEL_C  if width < min_cols                 ("a limited number of columns"),
 *   LU_LEVEL_A  else if sub <= max_sub_a * width    ("very few associated sub-columns"),
 *   LU_LEVEL_B  otherwise                           (many columns, many sub-columns).
 * min_cols <= 0 => the device's SM count (fewer columns than SMs cannot fill the GPU with one
 * CTA per column); max_sub_a <= 0 => 32 (one warp per sub-column fits one CTA per column).
 * d_row_ptr_lu / d_col_idx_lu: CSR of L+U, rows sorted; d_level[n]; d_type int32[num_levels];
 * d_sub int64[num_levels] or NULL.  Synchronises.  LU_ERR_ARG on null pointers / bad sizes.
 */
enum { LU_LEVEL_A = 0, LU_LEVEL_B = 1, LU_LEVEL_C = 2 };
lu_status lu_level_types(int32_t n, const int64_t *d_row_ptr_lu, const int32_t *d_col_idx_lu,
                         const int32_t *d_level, int32_t num_levels, int32_t min_cols,
                         int32_t max_sub_a, int32_t *d_type, int64_t *d_sub, void *stream);

/*
 * Numeric factorization (not part of the symbolic hot path) — Algorithm 2 of
 * PAPER.md, the hybrid column-based right-looking LU (L165-204), pivot-free (reading R29),
 * float values (the paper's precision).  As = "the non-zero filled-in matrix of A after
 * symbolic analysis" (L175) is stored in the CSR of L+U (d_row_ptr_lu int64[n+1],
 * d_col_idx_lu int32[nnz_lu], rows sorted, as lu_sym_emit writes them) as d_val_lu
 * float[nnz_lu], one value per pattern entry.
 *
 * lu_numeric_scatter: d_val_lu = A's values (d_val_a float[nnz_a], on A's CSR d_row_ptr_a /
 *   d_col_idx_a) at their L+U positions, 0 at fill entries.  LU_ERR_INPUT if an entry of A is
 *   not in the pattern (the pattern is not A's L+U).  Synchronises.
 *
 * lu_numeric_factor: Algorithm 2 in place on d_val_lu: afterwards the strictly lower entries
 *   hold L (unit diagonal implied) and the upper entries, diagonal included, hold U, A = L U.
 *   Columns are processed level by level (L206-208) from the level schedule d_level_ptr
 *   int64[num_levels+1] / d_level_cols int32[n] (lu_level_schedule), which MUST come from
 *   lu_levelize with LU_DEP_GLU3: that rule makes every value a level reads final before the
 *   level starts (under LU_DEP_U alone a U row may still be updated while it is read).
 *   Columns of one level update shared sub-columns with float atomics, so the rounding order
 *   (not the arithmetic) may vary from run to run.  The diagonal of every column must be in
 *   the pattern and non-zero when its column is reached: else LU_ERR_INPUT ("zero pivot");
 *   an update outside the pattern (a pattern that is not closed under elimination) is also
 *   LU_ERR_INPUT.  Scratch (O(n + nnz(L)), plus a 16-byte-per-update position table when
 *   it fits 1 GiB) is allocated per call from the stream-ordered pool.  All levels run in one
 *   cooperative launch with a grid barrier per level; environment knobs for A/B runs (results
 *   unchanged): LUSYM_NUMERIC_LAUNCH_PER_LEVEL=1 (one launch per level),
 *   LUSYM_NUMERIC_TABLE=0 (no position table), LUSYM_NUMERIC_TABLE_GB=<budget>.
 *   Synchronises.
 */
lu_status lu_numeric_scatter(int32_t n, const int64_t *d_row_ptr_a, const int32_t *d_col_idx_a,
                             const float *d_val_a, const int64_t *d_row_ptr_lu,
                             const int32_t *d_col_idx_lu, int64_t nnz_lu, float *d_val_lu,
                             void *stream);
lu_status lu_numeric_factor(int32_t n, const int64_t *d_row_ptr_lu, const int32_t *d_col_idx_lu,
                            const int64_t *d_level_ptr, const int32_t *d_level_cols,
                            int32_t num_levels, float *d_val_lu, void *stream);

/*
 * lu_numeric_factor_ex: the same with the storage mode of As chosen (§3.4):
 *   LU_NUMERIC_SPARSE: As(i,k) located in the sorted row by rank / binary search (Alg. 6) —
 *                      what lu_numeric_factor does (one cooperative launch for all levels);
 *   LU_NUMERIC_DENSE:  GLU3.0's dense format: the target row of each update expanded into a
 *                      dense n-long position map, so As(i,k) is addressed directly; each
 *                      concurrent CTA needs n ints, so at most M = L / (n sizeof) of them
 *                      (L352), L = half the free HBM; one launch per level;
 *   LU_NUMERIC_AUTO:   the paper's switch (L372): dense iff n <= L / (TB_max sizeof(float)),
 *                      TB_max = SMs x resident CTAs per SM; else sparse.
 * The results agree up to the float rounding order of the atomic updates.
 */
enum { LU_NUMERIC_AUTO = 0, LU_NUMERIC_DENSE = 1, LU_NUMERIC_SPARSE = 2 };
lu_status lu_numeric_factor_ex(int32_t n, const int64_t *d_row_ptr_lu,
                               const int32_t *d_col_idx_lu, const int64_t *d_level_ptr,
                               const int32_t *d_level_cols, int32_t num_levels, int32_t mode,
                               float *d_val_lu, void *stream);

/*
 * Row sharding with deferred rows (LU_F_DEFER_GLOBAL; reading G8).
 *
 * lu_sym_deferred_flags: d_flags[i] = 1 (int32[n], other entries untouched) for every row the
 *   last lu_sym_count call on this handle deferred.  The ranks' flags are OR-ed (all-reduced)
 *   by the caller.
 *
 * lu_sym_merge_deferred: finish the flagged rows (d_flags[i] != 0, ascending) by the row-merge
 *   closure over the complete pattern of every other row, given as the assembled CSR
 *   d_row_ptr_lu / d_col_idx_lu (rows sorted; flagged rows empty; d_fill_count[i] = their row
 *   lengths, 0 for flagged rows).  On return d_fill_count[i] holds every row's count,
 *   d_row_ptr_lu the final offsets and *nnz_lu (host) the final nnz; the handle's staging pool
 *   holds every row, so a following lu_sym_emit(h, 0, n, d_row_ptr_lu, new array, cap) writes
 *   the final CSR (the caller allocates it with the new nnz).  Every rank may run it on the
 *   same inputs: the result is identical.  LU_ERR_NOMEM if the staging pool cannot hold the
 *   assembled pattern plus n entries per flagged row.  Synchronises.
 */
lu_status lu_sym_deferred_flags(lu_sym *h, int32_t *d_flags, void *stream);
lu_status lu_sym_merge_deferred(lu_sym *h, const int32_t *d_flags, int32_t *d_fill_count,
                                int64_t *d_row_ptr_lu, const int32_t *d_col_idx_lu,
                                int64_t *nnz_lu, void *stream);

/* Copy the handle's statistics to *out (host). */
lu_status lu_sym_get_stats(const lu_sym *h, lu_sym_stats *out);

/*
 * Diagnostics (the paper's Fig. 3 per-row frontier profile, L249/L272): with d_prof != NULL
 * (device int64[4 n], borrowed) every later lu_sym_count records, for each row i it processes,
 * d_prof[4i+0] = SM clock cycles spent on the row, [4i+1] = vertices scanned, [4i+2] = BFS runs
 * (non-simple thresholds), [4i+3] = threshold windows.  NULL switches recording off.
 */
lu_status lu_sym_set_row_profile(lu_sym *h, int64_t *d_prof);

/* Free the handle's scratch (synchronises its streams).  NULL is a no-op. */
void lu_sym_destroy(lu_sym *h);

/* Static description of a status code. */
const char *lu_status_str(lu_status s);

/* Message of the last failing call on the calling host thread ("" if none). */
const char *lu_last_error(void);

/*
 * Environment knobs of the symbolic phase (A/B experiments and diagnostics; none changes a
 * result, DESIGN.md §5.1 has the measurements).  Read at lu_sym_create unless noted.
 *   LUSYM_TIGHT_CLASSES=0     row classes by halving the shared visited map (default: the largest
 *                             map that adds rows per SM, G5)
 *   LUSYM_ASYNC_OCC=<k>       barrier-free BFS (bfs_async) in classes of at most k rows per SM
 *                             (default 0: off; LU_F_ASYNC_BFS forces it); LUSYM_ASYNC_KEEP,
 *                             LUSYM_ASYNC_SLEEP its donation threshold and idle poll (ns)
 *                             (read once per process)
 *   LUSYM_MERGE_GRID_HEAD=<k> the whole grid finishes the first k deferred rows (default 2),
 *                             the clusters the rest; LUSYM_MERGE_GRID_MAX=<k> the whole list
 *                             when it has at most k rows (default 0)
 *   LUSYM_MERGE_CLUSTER=<g>   CTAs per deferred row in the tail (default 4; 1 = no cluster);
 *                             LUSYM_MERGE_HBM_BITMAP, LUSYM_MERGE_NOFILTER variants
 *   LUSYM_HEAVY_TOP=<k>       the last k rows in the shared-map class next to the sparse class
 *                             (default 0; LUSYM_HEAVY_GRID its rows in flight) (read once)
 *   LUSYM_DEFER_WINDOWS, LUSYM_SPARSE_DEFER_WINDOWS, LUSYM_FORCE_SPARSE, LUSYM_TOP_LBW
 *                             deferral thresholds and planner test knobs
 *   LUSYM_DEBUG_PLAN=1        print the row classes; LUSYM_DEBUG_CREATE=1 host time per create
 *                             step (read once)
 *   LUSYM_LIB=<path>          (Python binding) load another build of this library
 */

#ifdef __cplusplus
}
#endif

#endif /* LU_SYM_H */
