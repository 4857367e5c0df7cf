// Internal declarations shared by the CUDA translation units of liblusym.so.
// Nothing here is part of the public ABI (include/lu_sym.h is).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

// XOR swizzle of the shared visited words inside groups of 32 (fill2_impl.cuh phys); the host
// needs it too, for the encoded adjacency (encode_ell)
#ifndef LUSYM_SWZ
#define LUSYM_SWZ 1
#endif

namespace lusym {

// Traversal adjacency entry marking a vertex whose off-diagonal degree exceeds the ELL width:
// slot 0 = kHeavy, slot 1 = row length, slots 2..3 = int64 offset of the row in A's col_idx.
constexpr int32_t kHeavy = INT32_MIN;
constexpr int kHdrBytes = 1024;   // per-CTA shared header (scalars + scan scratch)

// Device-side statistics slots (unsigned long long each).
enum StatSlot { kStatEdges = 0, kStatVerts = 1, kStatSpills = 2, kStatErr = 3, kStatCount = 4 };

struct Fill2Params {
    int32_t n;
    const int64_t *rp;        // A row_ptr [n+1]
    const int32_t *ci;        // A col_idx
    const int32_t *ell;       // traversal adjacency, n x W int32 (16 B aligned)
    const int32_t *elle;      // ... the same with light neighbours encoded (enc_slot) for the
                              // shared-map kernels' BFS, or null
    int32_t row_begin, row_end;
    int32_t descending;       // 1: heaviest (largest id) first
    int32_t *fill_count;      // count pass
    const int64_t *rp_lu;     // emit pass
    int32_t *ci_lu;
    uint32_t *gbitmap;        // visited bitmaps in HBM (one slot per CTA) or null
    uint32_t *dbitmap;        // "threshold done" bitmaps in HBM (one slot per CTA)
    int64_t gbitmap_stride;   // words per slot
    int32_t *gspill;          // frontier spill, 2 x spill_cap per CTA
    int64_t spill_cap;
    int32_t nw;               // visited words held in shared memory (whole swizzle groups)
    int32_t lbw;              // kVisSplit: words [0, lbw) are in shared memory
    int32_t sw;               // summary words = ceil(nw/32) (shared memory)
    int32_t q;                // shared frontier capacity per buffer (entries)
    int32_t wcap;             // window capacity (<= q); 1 = one threshold at a time
    unsigned long long *row_counter;
    unsigned long long *stats;  // kStatCount slots
    // rows taken from row_list[0..list_len) instead of [row_begin, row_end) when non-null
    const int32_t *row_list;
    int32_t list_len;
    // staging (kStage): per-CTA L buffer (spill_cap entries), pool, per-row pool offset
    int32_t *stg;
    int32_t *pool;
    int64_t pool_cap;
    int64_t *row_off;
    unsigned long long *pool_cursor;
    int32_t *unstaged;
    unsigned long long *unstaged_cnt;
    // optional per-row profile (4 x int64 per row: cycles, vertices scanned, BFS runs, windows)
    int64_t *row_prof;
    // self-continuation rounds per BFS level (scan_level); 0 = plain level-synchronous BFS
    int32_t kloc;
    // count the traversed edges of light vertices too (exact TE, reading R24; ~W+2 integer
    // instructions per scanned vertex, so only when LU_F_COUNT_TE asks for it)
    int32_t count_te = 0;
    // row_list length read on the device (a list built by an earlier kernel), when non-null
    const unsigned long long *list_len_dev = nullptr;
    // kStage: entries <= i of each staged row (L part + diagonal), for the row-merge tail
    int32_t *ucut = nullptr;
    // deferral (kStage, reading G8): a row i >= defer_from whose threshold loop reaches
    // defer_win + 1 windows is abandoned and listed (at most defer_max rows) for the
    // row-merge tail; defer_win = 0 disables it
    int32_t defer_win = 0, defer_from = 0, defer_max = 0;
    int32_t *defer_list = nullptr;
    unsigned long long *defer_cnt = nullptr;
    // below-threshold traversal without level barriers (bfs_async): ring entries per warp in
    // the frontier queues' shared memory (a power of two >= 64); 0 = level-synchronous BFS
    int32_t aring = 0;
    int32_t akeep = 32;    // bfs_async: entries a warp keeps when it donates to idle warps
    int32_t asleep = 1500; // bfs_async: ns an idle warp sleeps between polls of the pool
};
enum Fill2Mode { kCount = 0, kEmit = 1, kStage = 2 };
// row_off value of a row deferred to the row-merge tail and not finished yet
constexpr int64_t kRowDeferred = -2;

// merge_kernels.cu — deferred rows by row-merge closure over staged rows (reading G8)
struct MergeParams {
    int32_t n;
    const int64_t *rp;                 // A
    const int32_t *ci;
    int32_t *pool;                     // staging pool (read: rows t < i; written: row i)
    int64_t pool_cap;
    unsigned long long *pool_cursor;
    int64_t *row_off;                  // [n] pool offset, -1 unstaged, kRowDeferred pending
    int32_t *ucut;                     // [n] entries <= t of staged row t
    int32_t *fill_count;               // [n]
    const int32_t *list;               // deferred rows, ascending, list_cnt[0] (<= list_max)
    const unsigned long long *list_cnt;
    int32_t list_max;
    unsigned long long *counter;       // row claims
    uint32_t *gbitmap;                 // per-CTA visited slot (when not in shared memory)
    int64_t gb_stride;
    int32_t *spill;                    // per CTA: 2 x spill_cap frontier entries
    int64_t spill_cap;
    int32_t *wait;                     // per CTA: list_max deferred rows waited on
    int32_t *fail_list;                // rows the tail could not finish (-> fill2 fallback)
    unsigned long long *fail_cnt;
    unsigned long long *stats;         // [0] U entries read, [1] rounds, [2] waits
    int32_t q;                         // shared frontier capacity per buffer
    int32_t cl_filter = 0;             // cluster mode: words of the per-CTA filter (0: none)
    // grid-wide mode (k_merge_grid): the whole GPU finishes the deferred rows one at a time in
    // increasing order when there are at most grid_max of them (0: never)
    int32_t grid_max = 0;
    int32_t grid_head = 0;             // > 0: the grid takes the first grid_head rows of any list
    uint32_t *gbits = nullptr;         // [ceil(n/32)] visited bitmap of the row in progress
    int32_t *gq = nullptr;             // [2 n] frontier buffers
    long long *glen = nullptr;         // [n] U segment length of each frontier member
    long long *goff = nullptr;         // [n] its pool offset
    long long *gstart = nullptr;       // [n + 64] flat start of each non-empty segment (compacted)
    long long *gcoff = nullptr;        // [n] its pool offset (compacted)
    long long *gpart = nullptr;        // [4 * grid + 8] per-CTA partial sums, the row's pool offset
    int32_t *gctrl = nullptr;          // [16] counters
    int32_t grid_filter = 0;           // shared-memory filter words per CTA (0: none)
};
// mode 0: one CTA per row, bitmap in shared memory; 1: one CTA, bitmap in an HBM slot;
// 2: a cluster of g CTAs per row, bitmap sliced over their shared memories (DSMEM)
size_t merge_smem_bytes(int n, int mode, int g, int q, bool filter = false);
cudaError_t merge_configure(size_t smem);
cudaError_t merge_max_clusters(int g, size_t smem, int *clusters);
// sort list[0..min(*cnt, max)) ascending (one CTA; max <= 4096)
cudaError_t merge_sort_list(int32_t *list, const unsigned long long *cnt, int32_t max,
                            cudaStream_t s);
cudaError_t merge_launch(const MergeParams &p, int mode, int g, int grid, size_t smem,
                         cudaStream_t s);
// the grid-wide mode: one cooperative launch of *grid CTAs (set by merge_grid_size); it does
// nothing when the list holds more than p.grid_max rows, else it finishes them all and marks
// the list claimed so that the cluster kernel launched after it exits at once
cudaError_t merge_grid_size(int n, int *grid, int *filter_words);
cudaError_t merge_grid_launch(const MergeParams &p, int grid, cudaStream_t s);
// row sharding with deferred rows (LU_F_DEFER_GLOBAL)
cudaError_t zero_deferred_counts(const int32_t *list, const unsigned long long *cnt, int32_t max,
                                 int32_t *fill_count, cudaStream_t s);
cudaError_t deferred_to_flags(const int32_t *list, const unsigned long long *cnt, int32_t max,
                              int32_t *flags, cudaStream_t s);
// row_off / ucut of the assembled CSR (flagged rows: kRowDeferred); list[flag_pos[i]] = i for
// flagged rows (flag_pos = exclusive prefix sum of flags: ascending)
cudaError_t prep_merge(int32_t n, const int32_t *flags, const int64_t *rp, const int32_t *ci,
                       int64_t *row_off, int32_t *ucut, const int64_t *flag_pos, int32_t *list,
                       cudaStream_t s);
constexpr int kMergeNT = 1024;
constexpr int kMergeSortMax = 4096;

// Visited storage of a row in flight (frontiers are lists in shared memory, spilling to HBM).
//   kVisSmem   : visited bitmap in shared memory
//   kVisGlobal : visited bitmap in an HBM slot per CTA (n too large for shared memory)
//   kVisSplit  : words [0, lbw) in shared memory, the rest in the HBM slot (row classes)
enum Fill2Vis { kVisSmem = 0, kVisGlobal = 1, kVisSplit = 2 };

// Stream-ordered device allocations from the current device's default memory pool, whose
// release threshold is raised once so that memory freed by one handle stays reserved for the
// next (creating and destroying handles then costs no cudaMalloc/cudaFree).  lu_sym_api.cu.
cudaError_t dev_alloc(void **p, size_t bytes, cudaStream_t s);
void dev_free(void *p, cudaStream_t s);

// fill2_kernels.cu (host dispatch; kernels instantiated in fill2_nt*.cu)
bool fill2_smem_base_ok(int dev);
size_t fill2_smem_bytes(int n, int smem_words, int q);
cudaError_t fill2_configure(int nt, int w, int vis, size_t smem);
cudaError_t fill2_occupancy(int nt, int w, int vis, size_t smem, int *occ);
cudaError_t fill2_launch(const Fill2Params &p, int nt, int w, int mode, int vis, int grid,
                         size_t smem, cudaStream_t s);
template <int NT>
cudaError_t fill2_launch_nt(const Fill2Params &p, int w, int mode, int vis, int grid, size_t smem,
                            cudaStream_t s);
template <int NT>
cudaError_t fill2_configure_nt(int w, int vis, size_t smem);
template <int NT>
cudaError_t fill2_occupancy_nt(int w, int vis, size_t smem, int *occ);

// prep_kernels.cu
cudaError_t validate_csr(int32_t n, int64_t nnz, const int64_t *rp, const int32_t *ci,
                         int64_t *d_bad /*[2]: first bad row, code*/, cudaStream_t s);
cudaError_t count_light(int32_t n, const int64_t *rp, const int32_t *ci, int w,
                        unsigned long long *d_cnt, cudaStream_t s);
cudaError_t build_ell(int32_t n, const int64_t *rp, const int32_t *ci, int w, int32_t *ell,
                      cudaStream_t s);
// the encoded copy for the shared-map kernels: light slots v -> phys(v >> 5) << 7 | (v & 31)
// (phys = the XOR swizzle of fill2_impl.cuh when swz), heavy records unchanged
cudaError_t encode_ell(int32_t n, int w, bool swz, const int32_t *ell, int32_t *elle,
                       cudaStream_t s);
// row_ptr[0..n] = exclusive prefix sum of counts[0..n); chained: offsets start at the value
// row_ptr[0] holds on entry (a row block continuing an earlier one), else at 0
cudaError_t scan_counts(int32_t n, const int32_t *counts, int64_t *row_ptr, int64_t *blk,
                        cudaStream_t s, bool chained = false);
size_t scan_scratch_elems(int32_t n);
cudaError_t count_far_entries(int32_t n, const int64_t *rp, const int32_t *ci, int32_t bound,
                              unsigned long long *d_cnt, cudaStream_t s);

// bound_kernels.cu — a-priori capacity of L+U from A (Theorem 1 row envelopes); synchronises
cudaError_t nnz_upper_bound(int32_t n, const int64_t *rp, const int32_t *ci, int64_t *h_bound,
                            cudaStream_t s);

// place_kernels.cu — symbolic_2 for staged rows: copy pool rows to their CSR slots
cudaError_t place_rows(int32_t row_begin, int32_t row_end, const int64_t *rp_lu,
                       const int64_t *row_off, const int32_t *pool, int32_t *ci_lu,
                       int64_t base, int64_t total, cudaStream_t s);
// rows of [row_begin, row_end) with row_off < 0 -> list[0..*cnt)
cudaError_t collect_unstaged(int32_t row_begin, int32_t row_end, const int64_t *row_off,
                             int32_t *list, unsigned long long *cnt, cudaStream_t s);

// schedule_kernels.cu — columns grouped by level (Fig. 1(d) form)
cudaError_t level_types(int32_t n, const int64_t *rp, const int32_t *ci, const int32_t *level,
                        int32_t num_levels, int32_t min_cols, int32_t max_sub_a, int32_t *type,
                        int64_t *sub, cudaStream_t s);
cudaError_t level_schedule(int32_t n, const int32_t *level, int32_t num_levels,
                           int64_t *level_ptr, int32_t *level_cols, int *h_bad, cudaStream_t s);
// a level schedule (level_ptr / cols) is a permutation of [0, n) under which every strict entry
// (i,j) of the pattern has level(min(i,j)) < level(max(i,j)) (the GLU3 rule); *h_bad = 1 if not
cudaError_t validate_schedule(int32_t n, const int64_t *rp, const int32_t *ci,
                              const int64_t *level_ptr, int32_t num_levels, const int32_t *cols,
                              int *h_bad, cudaStream_t s);

// numeric_kernels.cu — Algorithm 2 (numeric LU) on the L+U pattern, SURVEY 8(f4)
cudaError_t numeric_scatter(int32_t n, const int64_t *rpa, const int32_t *cia, const float *va,
                            const int64_t *rp, const int32_t *ci, int64_t nnz_lu, float *val,
                            int *h_err, cudaStream_t s);
cudaError_t numeric_factor(int32_t n, const int64_t *rp, const int32_t *ci,
                           const int64_t *h_level_ptr, const int64_t *level_ptr_d,
                           const int32_t *level_cols,
                           int32_t num_levels, int32_t num_sms, float *val, int *h_err,
                           cudaStream_t s, int dense_ctas = 0);

// levelize_kernels.cu
struct LevelizeScratch {
    int64_t *ustart = nullptr;  // [n] first strict-U position of row i
    int64_t *uend = nullptr;    // [n] end of the (pruned) successor range of row i
    int32_t *indeg = nullptr;   // [n]
    int32_t *queue = nullptr;   // [2n]
    int64_t *lt_ptr = nullptr;  // [n+1]  (GLU3 rule: transpose of strict L)
    int32_t *lt_idx = nullptr;  // [nnz_l]
    int64_t *lt_fill = nullptr; // [n] scatter cursors
    int64_t *scan_blk = nullptr;
    int32_t *ctrl = nullptr;    // device control block
    int32_t *chain = nullptr;   // [12n] J0 D0 J1 D1 nxt tail len best, then 16n bytes of
                                // per-head successor ranges
    int32_t n_cap = 0;
    int64_t lt_cap = 0;
};
struct LevelizeInfo {
    int32_t num_levels = 0, rounds = 0, wide_rounds = 0, narrow_rounds = 0, rank_rounds = 0;
    int32_t launches = 0;
};
cudaError_t levelize_run(int32_t n, const int64_t *rp_lu, const int32_t *ci_lu, int rule,
                         bool prune, bool contract, bool wide_only, LevelizeScratch &scr,
                         int32_t *level, LevelizeInfo *info, cudaStream_t s, const char **err);
void levelize_free(LevelizeScratch &scr, cudaStream_t s);

}  // namespace lusym
