// C ABI of liblusym.so (declared in include/lu_sym.h): handle, out-of-core planner, calls.
#include "lu_sym.h"
#include "internal.h"

#include <nvtx3/nvtx3.hpp>  // header-only: a named range per ABI call (for nsys / ncu)

#include <chrono>
#include <mutex>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include <cstring>
#include <string>
#include <utility>
#include <vector>

using namespace lusym;

namespace lusym {

cudaError_t dev_alloc(void **p, size_t bytes, cudaStream_t s)
{
    static bool configured[64] = {};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev >= 0 && dev < 64 && !configured[dev]) {
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t thr = UINT64_MAX;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        }
        configured[dev] = true;
    }
    return cudaMallocAsync(p, bytes, s);
}

void dev_free(void *p, cudaStream_t s)
{
    if (p) cudaFreeAsync(p, s);
}

}  // namespace lusym

namespace {

thread_local std::string g_err;

lu_status fail(lu_status s, const char *fmt, ...)
{
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_err = buf;
    return s;
}

#define CK(x)                                                                                \
    do {                                                                                     \
        cudaError_t e_ = (x);                                                                \
        if (e_ != cudaSuccess)                                                               \
            return fail(e_ == cudaErrorMemoryAllocation ? LU_ERR_NOMEM : LU_ERR_CUDA,        \
                        "%s: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__);   \
    } while (0)

enum { kEvCount = 0, kEvScan = 1, kEvEmit = 2, kEvLev = 3, kEvTail = 4, kEvN = 5 };
constexpr int kSparseDeferWindows = 1024;  // sparse class (G9): see the comment in plan()
enum { kSlotPoolCursor = 9, kSlotUnstaged = 10, kSlotList = 11, kSlotClassCounter = 16,
       kSlotSetStride = 32, kSlotDefer = 112 /* [0] deferred rows, [1] tail claims,
       [2] failed rows, [3..5] tail statistics */, kStatSlots = 128, kMaxChunks = 64, kSets = 3 };

}  // namespace

struct RowClass {
    int32_t lo, hi;   // rows [lo, hi)
    int vis;          // kVisSmem / kVisGlobal / kVisSplit
    int smem_words;   // visited words held in shared memory
    int lbw;          // kVisSplit: words [0, lbw) in shared memory
    int nt, q, occ;
    size_t smem;
    int64_t cap = 0;  // per-CTA spill / staging capacity (entries)
    int grid = 0;
    int defer_win = 0;  // > 0: this class's own deferral threshold (windows), else the handle's
    // this class's disjoint scratch regions (classes run concurrently)
    int64_t spill_off = 0, stg_off = 0, map_off = 0;
    cudaStream_t stream = nullptr;  // classes after the first run on their own stream
    cudaEvent_t done = nullptr;
};

struct lu_sym {
    // grid-wide tail (k_merge_grid) for lists of at most mg_max deferred rows
    int mg_max = 0, mg_head = 0, mg_grid = 0, mg_filter = 0;
    uint32_t *mg_bits = nullptr;
    int32_t *mg_q = nullptr, *mg_ctrl = nullptr;
    long long *mg_ll = nullptr;
    int32_t n = 0;
    int64_t nnz_a = 0;
    const int64_t *rp = nullptr;
    const int32_t *ci = nullptr;
    lu_sym_opts opts;
    int device = 0;
    // traversal adjacency
    int32_t *ell = nullptr;
    int32_t *elle = nullptr;  // encoded copy (shared-map BFS), n <= 2^21 only
    int w = 8;
    // plan
    bool gb = false;
    int vis = kVisSmem;
    int nt = 256, q = 2048, grid = 0;
    size_t smem = 0;
    uint32_t *gbitmap = nullptr;
    uint32_t *dbitmap = nullptr;
    int64_t gb_stride = 0;
    int64_t map_words = 0;  // words of the HBM visited / done maps (all classes)
    int32_t *gspill = nullptr;
    int64_t spill_cap = 0;
    unsigned long long *dstats = nullptr;  // [0] row counter, [1..4] count pass, [5..8] emit,
                                           // [9] pool cursor, [10] unstaged rows, [11] list n
    int64_t *scan_blk = nullptr;
    int64_t *dbad = nullptr;
    uint64_t budget = 0;
    // staging (count writes every row to the pool; emit places it)
    bool staging = true;
    int32_t *stg = nullptr;      // per CTA: L entries of the row in flight (spill_cap each)
    int32_t *pool = nullptr;
    int64_t pool_cap = 0;        // entries; -1 = no pool could be allocated
    int64_t *row_off = nullptr;  // [n] pool offset of each staged row, -1 = not staged
    int32_t *unstaged = nullptr; // [n] rows that overflowed the pool / row list for re-traversal
    std::vector<RowClass> classes;  // Alg. 4 row classes, top (heaviest) first
    std::vector<std::pair<int32_t, int32_t>> staged;  // row ranges staged since the last reset
    // state
    bool scanned = false;
    int64_t nnz_lu = 0;
    lu_sym_stats stats;
    LevelizeScratch lev;
    cudaEvent_t ev[kEvN][2] = {};
    bool ev_used[kEvN] = {};
    int64_t scratch_bytes = 0;
    int64_t launches = 0;
    int64_t *row_prof = nullptr;  // borrowed, set by lu_sym_set_row_profile
    cudaStream_t stream = nullptr;  // stream of the last call (scratch is freed on it)
    std::vector<void *> managed;    // LU_F_MANAGED scratch (freed with cudaFree)
    // extra traversal scratch sets 1..kSets-1 (lu_sym_run_host: the heaviest row chunk on set
    // 0 while the others alternate on sets 1 and 2, so a chunk's CTAs take over the SMs the
    // previous one leaves while it drains); allocated on first use
    int32_t *gspillS[kSets] = {}, *stgS[kSets] = {};
    uint32_t *gbitmapS[kSets] = {}, *dbitmapS[kSets] = {};
    std::vector<cudaStream_t> cls_streamS[kSets];
    std::vector<cudaEvent_t> cls_doneS[kSets];
    cudaStream_t pipe_stream[4] = {};  // lu_sym_run_host: count streams of sets 1/2, place, copy
    cudaEvent_t pipe_ev[4][kMaxChunks + 1] = {};  // count done, scanned, placed, copied
    int64_t *pin = nullptr;                       // pinned host slot (chunk end offset)
    std::vector<int32_t> chunk_bounds;            // lu_sym_run_host row chunks (cached)
    bool heavy_last = false;                      // ... and whether the last chunk goes first
    // deferred rows (reading G8): fill2 abandons a row after defer_win threshold windows; the
    // row-merge tail (merge_kernels.cu) finishes it from the staged rows below it
    int32_t *ucut = nullptr;       // [n] entries <= i of each staged row
    int defer_win = 512, defer_max = 1024;
    bool defer_active = false;     // the pass being launched may defer rows >= defer_from
    int32_t defer_from = 0;
    int32_t *defer_list = nullptr, *fail_list = nullptr;  // [defer_max] each
    int32_t *mspill = nullptr, *mwait = nullptr;
    uint32_t *mgbitmap = nullptr;
    int merge_grid = 0, merge_q = 2048, merge_mode = 0, merge_g = 1, merge_filter = 0;
    bool merge_smem_bm = true;
    size_t merge_smem = 0;
    bool tail_ran = false;
    bool deferred_pending = false;  // LU_F_DEFER_GLOBAL count deferred rows, no tail yet
    double sparse_sv = -1;         // planner sample: mean SV per row (-1: not sampled)
};

namespace {

lu_status check_device(const lu_sym *h)
{
    int d = -1;
    CK(cudaGetDevice(&d));
    if (d != h->device)
        return fail(LU_ERR_STATE, "handle created on device %d, current device is %d", h->device,
                    d);
    return LU_OK;
}

template <class T>
lu_status dalloc(lu_sym *h, T **p, size_t elems)
{
    size_t bytes = elems * sizeof(T);
    if (bytes == 0) bytes = 16;
    cudaError_t e = dev_alloc(reinterpret_cast<void **>(p), bytes, h->stream);
    if (e != cudaSuccess)
        return fail(LU_ERR_NOMEM, "cudaMalloc(%zu bytes): %s", bytes, cudaGetErrorString(e));
    h->scratch_bytes += (int64_t)bytes;
    return LU_OK;
}

bool is_managed(const lu_sym *h) { return (h->opts.flags & (LU_F_MANAGED | LU_F_MANAGED_PREFETCH)) != 0; }

// Traversal scratch: device memory from the stream-ordered pool, or (LU_F_MANAGED, the
// unified-memory variant of PAPER.md L237-239) cudaMallocManaged pages that migrate on first
// touch, optionally advised to and prefetched onto this GPU (LU_F_MANAGED_PREFETCH).
cudaError_t scratch_alloc_raw(lu_sym *h, void **p, size_t bytes)
{
    if (!is_managed(h)) return dev_alloc(p, bytes, h->stream);
    cudaError_t e = cudaMallocManaged(p, bytes, cudaMemAttachGlobal);
    if (e != cudaSuccess) return e;
    h->managed.push_back(*p);
    if (h->opts.flags & LU_F_MANAGED_PREFETCH) {
        cudaMemLocation loc;
        loc.type = cudaMemLocationTypeDevice;
        loc.id = h->device;
        if ((e = cudaMemAdvise(*p, bytes, cudaMemAdviseSetPreferredLocation, loc)) != cudaSuccess)
            return e;
        if ((e = cudaMemPrefetchAsync(*p, bytes, loc, 0, h->stream)) != cudaSuccess) return e;
    }
    return cudaSuccess;
}

template <class T>
lu_status salloc(lu_sym *h, T **p, size_t elems)
{
    if (!is_managed(h)) return dalloc(h, p, elems);
    size_t bytes = elems * sizeof(T);
    if (bytes == 0) bytes = 16;
    cudaError_t e = scratch_alloc_raw(h, reinterpret_cast<void **>(p), bytes);
    if (e != cudaSuccess)
        return fail(LU_ERR_NOMEM, "cudaMallocManaged(%zu bytes): %s", bytes, cudaGetErrorString(e));
    h->scratch_bytes += (int64_t)bytes;
    return LU_OK;
}

void free_handle(lu_sym *h)
{
    cudaStream_t s = h->stream;
    void *bufs[] = {h->ell,        h->elle,      h->gbitmap, h->dbitmap, h->gspill, h->dstats,
                    h->scan_blk,   h->dbad,      h->stg,     h->pool,   h->row_off,
                    h->unstaged,   h->ucut,      h->defer_list, h->fail_list, h->mspill,
                    h->mwait,      h->mgbitmap, h->mg_bits, h->mg_q, h->mg_ll, h->mg_ctrl};
    if (!h->managed.empty()) cudaStreamSynchronize(s);
    std::vector<void *> all(std::begin(bufs), std::end(bufs));
    for (int k = 1; k < kSets; ++k)
        for (void *b : {(void *)h->gspillS[k], (void *)h->stgS[k], (void *)h->gbitmapS[k],
                        (void *)h->dbitmapS[k]})
            all.push_back(b);
    for (void *b : all) {
        if (!b) continue;
        if (std::find(h->managed.begin(), h->managed.end(), b) != h->managed.end())
            cudaFree(b);
        else
            dev_free(b, s);
    }
    levelize_free(h->lev, s);
    for (auto &c : h->classes) {
        if (c.stream) cudaStreamDestroy(c.stream);
        if (c.done) cudaEventDestroy(c.done);
    }
    for (int k = 1; k < kSets; ++k) {
        for (auto cs : h->cls_streamS[k])
            if (cs) cudaStreamDestroy(cs);
        for (auto ce : h->cls_doneS[k])
            if (ce) cudaEventDestroy(ce);
    }
    for (auto ps : h->pipe_stream)
        if (ps) cudaStreamDestroy(ps);
    for (auto &row : h->pipe_ev)
        for (auto pe : row)
            if (pe) cudaEventDestroy(pe);
    if (h->pin) cudaFreeHost(h->pin);
    for (int k = 0; k < kEvN; ++k)
        for (int j = 0; j < 2; ++j)
            if (h->ev[k][j]) cudaEventDestroy(h->ev[k][j]);
    delete h;
}

// ---------------------------------------------------------------- out-of-core planner
// Paper (L239-243): chunk_size = L / (c n), c = 6 words per vertex per row in flight, and
// Alg. 4 (L272-277): the scratch a row needs grows with its id, so rows are split into ranges
// with different chunk sizes.  Here a row in flight is a CTA owning: a visited bitmap (shared
// memory when it fits, else an HBM slot), a level-1 summary, two shared frontier queues
// spilling to HBM.  Row classes: rows i < 32*lbw only need words [0, lbw) of the visited map in
// shared memory (their whole BFS region lies below i; marks above go to the HBM slot), so lower
// classes fit more rows per SM.  Within a class the CTA size and queue capacity maximise
// resident threads, then rows in flight; the HBM budget caps rows in flight.
#ifndef LUSYM_KLOC  // self-continuation rounds in latency-bound classes (scan_level)
#define LUSYM_KLOC 4
#endif
#ifndef LUSYM_KLOC_OCC  // ... those with at most this many rows per SM
#define LUSYM_KLOC_OCC 2
#endif

// classes with at most this many rows per SM run the asynchronous BFS (LUSYM_ASYNC_OCC: A/B)
const int g_async_occ = [] {
    const char *e = getenv("LUSYM_ASYNC_OCC");
    return e ? atoi(e) : 0;
}();

const int g_async_keep = [] {  // LUSYM_ASYNC_KEEP: A/B knob (entries kept when donating)
    const char *e = getenv("LUSYM_ASYNC_KEEP");
    return e ? std::max(1, std::min(atoi(e), 64)) : 32;
}();
const int g_async_sleep = [] {  // LUSYM_ASYNC_SLEEP: A/B knob (ns between pool polls)
    const char *e = getenv("LUSYM_ASYNC_SLEEP");
    return e ? atoi(e) : 1500;
}();

// LUSYM_HEAVY_TOP / LUSYM_HEAVY_GRID (A/B knobs): the last rows in a shared-map class next
// to the sparse class, and that class's rows in flight
const int g_heavy_top = [] {
    const char *e = getenv("LUSYM_HEAVY_TOP");
    return e ? atoi(e) : 0;
}();
const int g_heavy_grid = [] {
    const char *e = getenv("LUSYM_HEAVY_GRID");
    return e ? atoi(e) : 0;
}();

// class boundaries at the largest shared map that adds rows in flight (LUSYM_TIGHT_CLASSES=0:
// halve the map per class instead, round 1's ladder)
const bool g_tight_classes = [] {
    const char *e = getenv("LUSYM_TIGHT_CLASSES");
    return e ? atoi(e) != 0 : true;
}();

// Free device memory for the planner's budget.  cudaMemGetInfo takes from 0.1 ms to 95 ms
// (measured in bench.py's e2e loop, a create after another handle's destroy),
// so a reading younger than 30 s is reused per device.  The budget is 0.85 of it, the staging
// pool falls back to re-traversal if its allocation fails, and other allocations that still
// fail return LU_ERR_NOMEM.
cudaError_t mem_info(size_t *free_b, size_t *total_b)
{
    struct Reading {
        size_t free_b = 0, total_b = 0;
        std::chrono::steady_clock::time_point t;
        bool valid = false;
    };
    static Reading cache[64];
    static std::mutex mu;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const auto now = std::chrono::steady_clock::now();
    {
        std::lock_guard<std::mutex> lock(mu);
        if (dev >= 0 && dev < 64 && cache[dev].valid &&
            now - cache[dev].t < std::chrono::seconds(30)) {
            *free_b = cache[dev].free_b;
            *total_b = cache[dev].total_b;
            return cudaSuccess;
        }
    }
    e = cudaMemGetInfo(free_b, total_b);
    if (e == cudaSuccess && dev >= 0 && dev < 64) {
        std::lock_guard<std::mutex> lock(mu);
        cache[dev] = Reading{*free_b, *total_b, now, true};
    }
    return e;
}

// LUSYM_DEBUG_CREATE: host milliseconds of each create / plan step on stderr (diagnostic)
const bool g_dbg_create = getenv("LUSYM_DEBUG_CREATE") != nullptr;
std::chrono::steady_clock::time_point g_tc;
void dbg_lap(cudaStream_t s, const char *what)
{
    if (!g_dbg_create) return;
    cudaStreamSynchronize(s);
    const auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "lusym create: %-14s %8.3f ms\n", what,
            std::chrono::duration<double, std::milli>(now - g_tc).count());
    g_tc = now;
}

struct Cfg {
    int nt, q, occ;
    size_t smem;
    long key;
};

lu_status best_cfg(lu_sym *h, int smem_words, int vis, int smem_optin, Cfg *out, int want_nt = 0,
                   int min_q = 512)
{
    // kernel keys: CTA sizes 128..1024, and 1025 = 1024 threads with the one-CTA-per-SM
    // register budget (chosen on a tie, i.e. when shared memory allows one CTA per SM anyway)
    // (64: only on request — a sparse class or threads_per_row = 64)
    const int nts[6] = {64, 128, 256, 512, 1024, 1025};
    const int qs[6] = {128, 256, 512, 1024, 2048, 4096};
    Cfg best = {0, 0, 0, 0, -1};
    for (int a = 0; a < 6; ++a) {
        const int nt = nts[a];
        const int tpr = want_nt > 0 ? want_nt : h->opts.threads_per_row;
        if (tpr > 0 && nt != tpr && !(tpr == 1024 && nt == 1025)) continue;
        if (tpr <= 0 && nt == 64) continue;
        const int threads = nt > 1024 ? 1024 : nt;
        for (int b = 0; b < 6; ++b) {
            if (qs[b] < min_q && h->opts.queue_capacity <= 0) continue;
            int q = h->opts.queue_capacity > 0 ? h->opts.queue_capacity : qs[b];
            if (h->opts.queue_capacity > 0 && b > 0) break;
            if (q < 32) q = 32;
            const size_t smem = fill2_smem_bytes(h->n, smem_words, q);
            if (smem > (size_t)smem_optin) continue;
            // the attribute is a cap: set it to the device maximum so that every class sharing
            // this kernel can launch with its own dynamic shared memory size
            CK(fill2_configure(nt, h->w, vis, (size_t)smem_optin));
            int occ = 0;
            CK(fill2_occupancy(nt, h->w, vis, smem, &occ));
            if (occ < 1) continue;
            const long key = ((long)occ * threads << 24) | ((long)occ << 14) | q;
            if (key > best.key || (key == best.key && nt == 1025))
                best = Cfg{nt, q, occ, smem, key};
        }
    }
    *out = best;
    return LU_OK;
}

// Mean vertices scanned per row (SV, reading R24) over `cnt` rows evenly spread over [lo, hi),
// measured by running the count kernel on them with the configuration c (its own temporary
// scratch).  A row whose threshold chain exceeds 64 windows is abandoned where it stands
// (the circuit hubs would otherwise dominate the sample's time); its SV so far still counts.
lu_status sample_mean_sv(lu_sym *h, const RowClass &c, int32_t lo, int32_t hi, int cnt,
                         int sms, double *mean_sv)
{
    const int32_t n = h->n;
    cnt = std::max(1, std::min(cnt, hi - lo));
    std::vector<int32_t> rows((size_t)cnt);
    for (int k = 0; k < cnt; ++k)
        rows[(size_t)k] = lo + (int32_t)(((double)k + 0.5) * (hi - lo) / cnt);
    const int grid = std::min(cnt, sms * c.occ);
    const int64_t words = ((int64_t)n + 31) / 32 + 31;
    int32_t *d_rows = nullptr, *fc = nullptr, *spill = nullptr;
    uint32_t *dmap = nullptr, *gmap = nullptr;
    const size_t need = (size_t)cnt * 4 + (size_t)n * 4 + (size_t)grid * 2 * (size_t)n * 4 +
                        (size_t)grid * (size_t)words * 4 * (c.vis == kVisSmem ? 1 : 2);
    if (need > h->budget / 4) {  // never worth a large share of the budget
        *mean_sv = -1;
        return LU_OK;
    }
    cudaStream_t s = h->stream;
    CK(dev_alloc((void **)&d_rows, (size_t)cnt * 4, s));
    CK(dev_alloc((void **)&fc, (size_t)n * 4, s));
    CK(dev_alloc((void **)&spill, (size_t)grid * 2 * (size_t)n * 4, s));
    CK(dev_alloc((void **)&dmap, (size_t)grid * (size_t)words * 4, s));
    if (c.vis != kVisSmem) CK(dev_alloc((void **)&gmap, (size_t)grid * (size_t)words * 4, s));
    CK(cudaMemcpyAsync(d_rows, rows.data(), (size_t)cnt * 4, cudaMemcpyHostToDevice, s));
    unsigned long long *slots = h->dstats + kSlotDefer + 8;  // [0..3] stats, [4] row counter
    CK(cudaMemsetAsync(slots, 0, 5 * sizeof(unsigned long long), s));
    CK(cudaMemsetAsync(dmap, 0, (size_t)grid * (size_t)words * 4, s));
    if (gmap) CK(cudaMemsetAsync(gmap, 0, (size_t)grid * (size_t)words * 4, s));
    Fill2Params p;
    p.n = n;
    p.rp = h->rp;
    p.ci = h->ci;
    p.ell = h->ell;
    p.elle = h->elle;
    p.descending = 1;
    p.fill_count = fc;
    p.rp_lu = nullptr;
    p.ci_lu = nullptr;
    p.gbitmap = gmap;
    p.dbitmap = dmap;
    p.gbitmap_stride = words;
    p.gspill = spill;
    p.spill_cap = n;
    p.nw = c.smem_words;
    p.lbw = c.lbw;
    p.sw = (int32_t)((((int64_t)n + 31) / 32 + 31) / 32);
    p.q = c.q;
    p.wcap = c.q;
    p.row_counter = slots + 4;
    p.stats = slots;
    p.row_list = d_rows;
    p.list_len = cnt;
    p.row_begin = p.row_end = 0;
    p.stg = nullptr;
    p.pool = nullptr;
    p.pool_cap = 0;
    p.row_off = nullptr;
    p.pool_cursor = nullptr;
    p.unstaged = nullptr;
    p.unstaged_cnt = nullptr;
    p.row_prof = nullptr;
    p.kloc = c.occ <= LUSYM_KLOC_OCC ? LUSYM_KLOC : 0;
    p.defer_win = 64;
    p.defer_from = 0;
    CK(fill2_launch(p, c.nt, h->w, kCount, c.vis, grid, c.smem, s));
    h->launches += 1;
    unsigned long long st[kStatCount] = {};
    CK(cudaMemcpyAsync(st, slots, sizeof(st), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    for (void *b : {(void *)d_rows, (void *)fc, (void *)spill, (void *)dmap, (void *)gmap})
        dev_free(b, s);
    *mean_sv = (double)st[kStatVerts] / cnt;
    return LU_OK;
}

lu_status plan(lu_sym *h)
{
    int sms = 0, smem_optin = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device));
    CK(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, h->device));
    const int n = h->n;
    const int nw = (int)(((int64_t)n + 31) / 32);
    const int nw32 = (nw + 31) / 32 * 32;  // whole swizzle groups
    if (h->opts.threads_per_row > 0 && h->opts.threads_per_row != 128 &&
        h->opts.threads_per_row != 256 && h->opts.threads_per_row != 512 &&
        h->opts.threads_per_row != 1024 && h->opts.threads_per_row != 1025 &&
        h->opts.threads_per_row != 64)
        return fail(LU_ERR_ARG, "threads_per_row must be 64, 128, 256, 512, 1024 or 1025 (got %d)",
                    h->opts.threads_per_row);
    // top class: the whole visited map in shared memory, else in HBM
    Cfg cur;
    int vis = kVisGlobal, lbw = 0;
    lu_status st;
    // the shared-memory variants need the dynamic window at its usual base (fill2_impl.cuh)
    if (!fill2_smem_base_ok(h->device)) h->opts.flags |= LU_F_GLOBAL_BITMAP;
    if (!(h->opts.flags & LU_F_GLOBAL_BITMAP)) {
        if ((st = best_cfg(h, nw32, kVisSmem, smem_optin, &cur)) != LU_OK) return st;
        if (cur.key >= 0) {
            vis = kVisSmem;
            lbw = nw32;
        }
    }
    if (vis == kVisGlobal) {
        if ((st = best_cfg(h, 0, kVisGlobal, smem_optin, &cur)) != LU_OK) return st;
        if (cur.key < 0)
            return fail(LU_ERR_NOMEM, "no resident fill2 configuration (queue_capacity %d)",
                        h->opts.queue_capacity);
        lbw = nw32;  // for splitting below: start from the full map
    }
    if (const char *e = getenv("LUSYM_TOP_LBW")) {  // A/B knob: split the top class itself
        const int want = (atoi(e) + 31) / 32 * 32;
        Cfg c;
        if (want > 0 && want < nw32 &&
            (st = best_cfg(h, want, kVisSplit, smem_optin, &c)) == LU_OK && c.key >= 0) {
            cur = c;
            vis = kVisSplit;
            lbw = want;
        }
    }
    dbg_lap(h->stream, "plan: top cfg");
    // lower row classes (Alg. 4): shrink the shared part to the largest one that adds rows in
    // flight (a binary search over whole swizzle groups; or halve it), while that adds rows
    h->classes.clear();
    int hi = n;
    const bool one_class = (h->opts.flags & LU_F_ONE_CLASS) != 0;
    while (!one_class) {
        int nl = (lbw / 2 + 31) / 32 * 32;
        if (nl < 64 || nl >= lbw) break;
        Cfg c;
        if (g_tight_classes && vis != kVisGlobal && !(h->opts.flags & LU_F_FORCE_CLASSES)) {
            // the largest shared part (whole swizzle groups) that adds rows in flight, instead
            // of half of the current one (occupancy only grows as the part shrinks): cfg4
            // 8,505 -> 7,337 ms (profiles/r02/ab_tight_classes.log)
            int ulo = 2, uhi = lbw / 32 - 1, best_u = 0;
            while (ulo <= uhi) {
                const int um = (ulo + uhi) / 2;
                Cfg t;
                if ((st = best_cfg(h, um * 32, kVisSplit, smem_optin, &t)) != LU_OK) return st;
                if (t.key >= 0 && t.occ > cur.occ) {
                    best_u = um;
                    ulo = um + 1;
                } else {
                    uhi = um - 1;
                }
            }
            if (best_u) nl = best_u * 32;
        }
        if ((st = best_cfg(h, nl, kVisSplit, smem_optin, &c)) != LU_OK) return st;
        if (c.key < 0) {
            if (vis != kVisGlobal) break;
            lbw = nl;  // an HBM-resident top class: keep halving until a split map fits
            continue;
        }
        if (c.occ <= cur.occ && !(h->opts.flags & LU_F_FORCE_CLASSES)) break;
        if (!(h->opts.flags & LU_F_FORCE_CLASSES)) {
            // the new class's pattern marks above its shared part go to HBM atomics: split
            // only while they are under a quarter of its entries (grids: the k entries per
            // boundary row; ND-ordered circuits with hubs last: the hub and top-separator
            // incidences, ~8%; unordered random matrices: about half, so no split)
            unsigned long long far = 0, ent = 0;
            const int rows = nl * 32 < n ? nl * 32 : n;
            CK(count_far_entries(n, h->rp, h->ci, nl * 32, h->dstats + 14, h->stream));
            CK(cudaMemcpyAsync(&far, h->dstats + 14, 8, cudaMemcpyDeviceToHost, h->stream));
            CK(cudaMemcpyAsync(&ent, h->rp + rows, 8, cudaMemcpyDeviceToHost, h->stream));
            CK(cudaStreamSynchronize(h->stream));
            if (far * 4 > ent) break;
        }
        const int lo = nl * 32 < hi ? nl * 32 : hi;  // rows i < 32*nl fit the smaller map
        const int sw_words = vis == kVisSmem ? nw32 : (vis == kVisSplit ? lbw : 0);
        h->classes.push_back(RowClass{lo, hi, vis, sw_words, vis == kVisGlobal ? 0 : sw_words,
                                      cur.nt, cur.q, cur.occ, cur.smem});
        hi = lo;
        vis = kVisSplit;
        lbw = nl;
        cur = c;
    }
    {
        const int sw_words = vis == kVisSmem ? nw32 : (vis == kVisSplit ? lbw : 0);
        h->classes.push_back(RowClass{0, hi, vis, sw_words, vis == kVisGlobal ? 0 : sw_words,
                                      cur.nt, cur.q, cur.occ, cur.smem});
    }
    dbg_lap(h->stream, "plan: classes");
    size_t free_b = 0, total_b = 0;
    CK(mem_info(&free_b, &total_b));
    dbg_lap(h->stream, "plan: meminfo");
    const uint64_t budget = h->opts.scratch_budget_bytes ? h->opts.scratch_budget_bytes
                                                         : (uint64_t)(0.85 * (double)free_b);
    h->budget = budget;
    h->staging = !(h->opts.flags & LU_F_TWO_PASS);
    h->gb_stride = nw32;
    // Sparse rows (reading G9): where a class holds few rows per SM because its shared visited
    // map is large, but the rows visit only a small part of it (a sample's mean SV < n/16 —
    // ND-ordered circuits scan ~3K of 10^6 vertices per row, natural-order grids ~i), the
    // whole range is better served by HBM visited slots (L2-resident) and 64-thread CTAs at
    // 32 rows per SM: latency is hidden by rows in flight instead of threads per row (cfg3:
    // 1/2/4/8 rows per SM in four shared-map classes 630 ms, 16 rows of 128 threads 195 ms,
    // 32 rows of 64 threads 159 ms, scripts/exp_plan.py).
    h->sparse_sv = -1;
    if (!(h->opts.flags & (LU_F_ONE_CLASS | LU_F_GLOBAL_BITMAP | LU_F_FORCE_CLASSES |
                           LU_F_NO_SPARSE)) &&
        h->opts.threads_per_row == 0 && h->opts.queue_capacity == 0) {
        // (a shared window of 4-64 KB just below each row's own word, the rest in the HBM slot,
        // measured slower on cfg3 than no shared visited words: 148/153/185 ms against 146 —
        // the window costs rows per SM, profiles/r02/ab_window.log)
        Cfg g;
        // 128-entry queues: the shared header, summary and queues of a 64-thread CTA then take
        // 6 KB and 32 rows fit an SM (28 with 256 entries): cfg3 count 130 -> 124 ms
        // (profiles/r02/sparse_minq.log; LUSYM_SPARSE_MINQ: A/B knob)
        const char *mq = getenv("LUSYM_SPARSE_MINQ");
        if ((st = best_cfg(h, 0, kVisGlobal, smem_optin, &g, 64, mq ? atoi(mq) : 128)) != LU_OK)
            return st;
        size_t kc = 0;
        // candidates: the classes (from the top) with fewer rows per SM than the sparse class,
        // considered only when the top class's shared map holds it below 8 rows per SM
        while (g.key >= 0 && kc < h->classes.size() && h->classes[kc].occ < g.occ &&
               h->classes.front().occ < 8)
            ++kc;
        const bool force = getenv("LUSYM_FORCE_SPARSE") != nullptr;  // test knob
        if (force && g.key >= 0) kc = h->classes.size();
        if (kc > 0) {
            double sv = -1;
            const int32_t lo = h->classes[kc - 1].lo;
            if ((st = sample_mean_sv(h, h->classes[0], lo, n, 256, sms, &sv)) != LU_OK) return st;
            if (force) sv = 0;
            h->sparse_sv = sv;
            if (sv >= 0 && sv < (double)n / 16) {
                const RowClass top0 = h->classes.front();
                h->classes.erase(h->classes.begin(), h->classes.begin() + (long)kc);
                h->classes.insert(h->classes.begin(),
                                  RowClass{lo, n, kVisGlobal, 0, 0, g.nt, g.q, g.occ, g.smem});
                // 64 threads and 256-entry windows make each threshold window slow: abandon a
                // row (G8) after fewer windows than a shared-map class would
                h->classes.front().defer_win = kSparseDeferWindows;
                if (const char *e = getenv("LUSYM_SPARSE_DEFER_WINDOWS"))  // A/B knob
                    h->classes.front().defer_win = atoi(e);
                // heavy top rows (the last separators of a nested-dissection order scan a large
                // part of the graph): back to the shared-map top class (A/B knob)
                const int heavy = g_heavy_top;
                if (heavy > 0 && heavy < n - lo && top0.vis == kVisSmem) {
                    RowClass t = top0;
                    t.lo = n - heavy;
                    t.hi = n;
                    t.defer_win = h->classes.front().defer_win;
                    h->classes.front().hi = n - heavy;
                    h->classes.insert(h->classes.begin(), t);
                }
            }
        }
    }
    dbg_lap(h->stream, "plan: sparse");
    // HBM budget: everything the handle allocates stays within scratch_budget_bytes.
    // Per row in flight: frontier spill (2 x cap) + L staging (cap) + done map (+ the HBM
    // visited slot); cap = rows of the class (a row's frontier and L part lie below i).  Every
    // class gets one row in flight, then the rest of the budget goes to the classes in order,
    // top (heaviest rows) first; classes run concurrently on disjoint regions.
    const bool need_hbm_map = h->classes.front().vis != kVisSmem || h->classes.size() > 1;
    const uint64_t fixed = (uint64_t)n * 4 + (h->staging ? (uint64_t)n * 12 : 0);
    std::vector<uint64_t> per_row(h->classes.size());
    uint64_t min_total = fixed;
    for (size_t k = 0; k < h->classes.size(); ++k) {
        RowClass &c = h->classes[k];
        c.cap = c.hi > 0 ? c.hi : 1;
        per_row[k] = (uint64_t)(h->staging ? 3 : 2) * c.cap * 4 +
                     (uint64_t)(need_hbm_map ? 2 : 1) * h->gb_stride * 4;
        min_total += per_row[k];
    }
    const uint64_t used = (uint64_t)h->scratch_bytes;
    if (budget < used + min_total)
        return fail(LU_ERR_NOMEM, "scratch budget %llu B < %llu B (adjacency and statistics "
                    "%llu B + one row in flight per row class %llu B)",
                    (unsigned long long)budget, (unsigned long long)(used + min_total),
                    (unsigned long long)used, (unsigned long long)min_total);
    uint64_t have = budget - used - min_total;
    uint64_t need_spill = 0, need_stg = 0, need_map = 0;
    int max_grid = 0;
    for (size_t k = 0; k < h->classes.size(); ++k) {
        RowClass &c = h->classes[k];
        int64_t grid = (int64_t)sms * c.occ;
        if (h->opts.rows_in_flight > 0 && h->opts.rows_in_flight < grid)
            grid = h->opts.rows_in_flight;
        if (k == 0 && g_heavy_top > 0 && g_heavy_grid > 0 && h->classes.size() > 1 &&
            h->classes[1].vis == kVisGlobal && g_heavy_grid < grid)
            grid = g_heavy_grid;
        const int64_t extra = std::min<int64_t>(grid - 1, (int64_t)(have / per_row[k]));
        c.grid = (int)(1 + std::max<int64_t>(extra, 0));
        have -= (uint64_t)(c.grid - 1) * per_row[k];
        const int64_t cap = c.cap;
        c.spill_off = (int64_t)need_spill;
        c.stg_off = (int64_t)need_stg;
        c.map_off = (int64_t)need_map;
        need_spill += (uint64_t)2 * cap * c.grid;
        need_stg += (uint64_t)cap * c.grid;
        need_map += (uint64_t)h->gb_stride * c.grid;
        max_grid = std::max(max_grid, c.grid);
    }
    h->grid = max_grid;
    h->map_words = (int64_t)need_map;
    dbg_lap(h->stream, "plan: budget");
    if ((st = salloc(h, &h->gspill, need_spill)) != LU_OK) return st;
    if (need_hbm_map && (st = salloc(h, &h->gbitmap, need_map)) != LU_OK) return st;
    if ((st = salloc(h, &h->dbitmap, need_map)) != LU_OK) return st;
    for (size_t k = 0; k < h->classes.size(); ++k) {
        CK(cudaEventCreateWithFlags(&h->classes[k].done, cudaEventDisableTiming));
        if (k > 0) CK(cudaStreamCreateWithFlags(&h->classes[k].stream, cudaStreamNonBlocking));
    }
    if ((st = salloc(h, &h->unstaged, (size_t)n)) != LU_OK) return st;
    if (h->staging) {
        if ((st = salloc(h, &h->stg, need_stg)) != LU_OK) return st;
        if ((st = salloc(h, &h->row_off, (size_t)n)) != LU_OK) return st;
        if ((st = salloc(h, &h->ucut, (size_t)n)) != LU_OK) return st;
    }
    dbg_lap(h->stream, "plan: alloc");
    // deferred rows (reading G8)
    {
        const int dw = h->opts.defer_windows, dm = h->opts.defer_max;
        h->defer_win = (h->opts.flags & LU_F_NO_DEFER) || dw < 0 ? 0 : (dw > 0 ? dw : 4096);
        h->defer_max = dm > 0 ? std::min(dm, (int)kMergeSortMax) : 1024;
        if (const char *e = getenv("LUSYM_DEFER_WINDOWS")) h->defer_win = atoi(e);
        if (!h->staging) h->defer_win = 0;
    }
    if (getenv("LUSYM_DEBUG_PLAN")) {
        for (auto &c : h->classes)
            fprintf(stderr,
                    "lusym plan: rows [%d,%d) vis %d smem_words %d lbw %d nt %d q %d occ %d "
                    "smem %zu grid %d\n",
                    c.lo, c.hi, c.vis, c.smem_words, c.lbw, c.nt, c.q, c.occ, c.smem, c.grid);
    }
    // summary fields (the top class)
    const RowClass &top = h->classes.front();
    h->vis = top.vis;
    h->gb = top.vis == kVisGlobal;
    h->nt = top.nt;
    h->q = top.q;
    h->smem = top.smem;
    return LU_OK;
}

void ev_begin(lu_sym *h, int k, cudaStream_t s)
{
    if (!h->ev[k][0]) {
        cudaEventCreate(&h->ev[k][0]);
        cudaEventCreate(&h->ev[k][1]);
    }
    cudaEventRecord(h->ev[k][0], s);
}

void ev_end(lu_sym *h, int k, cudaStream_t s)
{
    cudaEventRecord(h->ev[k][1], s);
    h->ev_used[k] = true;
}

// One traversal pass over rows [rb, re) (or row_list): one launch per row class, top class
// (heaviest rows) first, as Alg. 4 launches each part in turn.
// set: traversal scratch set (0, or 1 = the second set of lu_sym_run_host); reset_stats: zero
// the pass statistics first (a pipelined run accumulates over its chunks).
lu_status run_pass(lu_sym *h, int mode, int32_t rb, int32_t re, int32_t *fill_count,
                   const int64_t *rp_lu, int32_t *ci_lu, cudaStream_t s,
                   const int32_t *row_list = nullptr, int32_t list_len = 0, int set = 0,
                   bool reset_stats = true, const unsigned long long *list_len_dev = nullptr)
{
    const bool emit = mode == kEmit;
    unsigned long long *st = h->dstats + (emit ? 5 : 1);
    int32_t *gspill = set ? h->gspillS[set] : h->gspill;
    int32_t *stg = set ? h->stgS[set] : h->stg;
    uint32_t *gbitmap = set ? h->gbitmapS[set] : h->gbitmap;
    uint32_t *dbitmap = set ? h->dbitmapS[set] : h->dbitmap;
    unsigned long long *counters = h->dstats + kSlotClassCounter + set * kSlotSetStride;
    if (reset_stats) CK(cudaMemsetAsync(st, 0, sizeof(unsigned long long) * kStatCount, s));
    if (gbitmap) CK(cudaMemsetAsync(gbitmap, 0, sizeof(uint32_t) * h->map_words, s));
    CK(cudaMemsetAsync(dbitmap, 0, sizeof(uint32_t) * h->map_words, s));
    CK(cudaMemsetAsync(counters, 0, sizeof(unsigned long long) * h->classes.size(), s));
    if (h->row_prof && mode != kEmit && !row_list)
        CK(cudaMemsetAsync(h->row_prof + 4 * (size_t)rb, 0,
                           sizeof(int64_t) * 4 * (size_t)(re - rb), s));
    Fill2Params p;
    p.n = h->n;
    p.rp = h->rp;
    p.ci = h->ci;
    p.ell = h->ell;
    p.elle = h->elle;
    p.descending = (h->opts.flags & LU_F_ASCENDING) ? 0 : 1;
    p.fill_count = fill_count;
    p.rp_lu = rp_lu;
    p.ci_lu = ci_lu;
    p.gbitmap_stride = h->gb_stride;
    p.sw = (int32_t)((((int64_t)h->n + 31) / 32 + 31) / 32);
    p.stats = st;
    p.pool = h->pool;
    p.pool_cap = h->pool_cap;
    p.row_off = h->row_off;
    p.pool_cursor = h->dstats + kSlotPoolCursor;
    p.unstaged = h->unstaged;
    p.unstaged_cnt = h->dstats + kSlotUnstaged;
    p.row_prof = h->row_prof;
    p.ucut = h->ucut;
    p.list_len_dev = list_len_dev;
    p.count_te = (h->opts.flags & LU_F_COUNT_TE) ? 1 : 0;
    if (mode == kStage && h->defer_active && !row_list) {
        p.defer_win = h->defer_win;
        p.defer_from = h->defer_from;
        p.defer_max = h->defer_max;
        p.defer_list = h->defer_list;
        p.defer_cnt = h->dstats + kSlotDefer;
    }
    // classes run concurrently: the top class on s, the others on their own streams forked
    // from s, so lower-class CTAs take over SMs as soon as top-class CTAs drain
    bool forked = false;
    for (size_t k = 0; k < h->classes.size(); ++k) {
        const RowClass &c = h->classes[k];
        if (p.defer_win > 0 && c.defer_win > 0) p.defer_win = std::min(h->defer_win, c.defer_win);
        else if (p.defer_win > 0) p.defer_win = h->defer_win;
        // a row list (rows that did not fit the staging pool) runs in the top class only
        if (row_list && k > 0) break;
        const int32_t lo = row_list ? 0 : std::max(rb, c.lo), hi = row_list ? 0 : std::min(re, c.hi);
        const int rows = row_list ? (list_len_dev ? c.grid : list_len) : hi - lo;
        if (rows <= 0) continue;
        cudaStream_t cs = s;
        if (k > 0) {
            cudaEvent_t fork_ev = set ? h->cls_doneS[set][0] : h->classes[0].done;
            if (!forked) {
                CK(cudaEventRecord(fork_ev, s));
                forked = true;
            }
            cs = set ? h->cls_streamS[set][k] : c.stream;
            CK(cudaStreamWaitEvent(cs, fork_ev, 0));
        }
        p.row_begin = lo;
        p.row_end = hi;
        p.row_list = row_list;
        p.list_len = list_len;
        p.spill_cap = c.cap;
        p.gspill = gspill + c.spill_off;
        p.stg = stg ? stg + c.stg_off : nullptr;
        p.gbitmap = gbitmap ? gbitmap + c.map_off : nullptr;
        p.dbitmap = dbitmap + c.map_off;
        p.row_counter = counters + k;
        p.nw = c.smem_words;
        p.lbw = c.lbw;
        p.q = c.q;
        p.wcap = (h->opts.flags & LU_F_NO_BATCH) ? 1 : c.q;
        // one row per SM, or a pass with at most two rows per CTA in flight (cfg1: 4,096 rows on
        // 2,368 CTAs): a BFS level is latency-bound, let lanes run ahead a little (cfg1 count
        // 0.328 -> 0.305 ms; with many rows per CTA the extra rounds cost issue slots: cfg2 and
        // cfg5 twice as slow, profiles/r02/knobs_sc.log)
        // (the class's whole row range, not this call's: a chunk of lu_sym_run_host is short)
        const bool few_rows = (int64_t)(c.hi - c.lo) <= 2 * (int64_t)c.grid;
        p.kloc = ((c.occ <= LUSYM_KLOC_OCC || few_rows || (h->opts.flags & LU_F_SELF_CONT)) &&
                  !(h->opts.flags & LU_F_NO_SELF_CONT))
                     ? LUSYM_KLOC
                     : 0;
        // rows with the SM (nearly) to themselves: BFS without level barriers (bfs_async),
        // its per-warp rings carved out of the class's two frontier queues
        // (compiled into the 1024-thread one-CTA-per-SM kernel only: at 32 registers per
        // thread it would spill in the other kernels' hot loops)
        p.aring = 0;
        if (c.nt == 1025 && !(h->opts.flags & LU_F_NO_ASYNC_BFS) &&
            (c.occ <= g_async_occ || (h->opts.flags & LU_F_ASYNC_BFS))) {
            const int nwarps = (c.nt > 1024 ? 1024 : c.nt) / 32;
            int r = 1024;
            while (r > c.q / nwarps) r >>= 1;  // rings: half the queues; pool: the rest
            if (r >= 64) p.aring = r;
            p.akeep = g_async_keep;
            p.asleep = g_async_sleep;
        }
        if ((h->opts.flags & LU_F_PAPER_CHUNKS) && !row_list) {
            // Alg. 3 / Alg. 4 as printed: chunk_size = L / (c n) rows per launch (c = 6 words of
            // 4 B per vertex, L = scratch budget, reading R16), launches in increasing row order
            const uint64_t per_row = (uint64_t)6 * 4 * (uint64_t)h->n;
            int64_t chunk = (int64_t)(h->budget / (per_row ? per_row : 1));
            if (chunk < 1) chunk = 1;
            for (int64_t c0 = lo; c0 < hi; c0 += chunk) {
                const int64_t c1 = std::min<int64_t>(hi, c0 + chunk);
                CK(cudaMemsetAsync(p.row_counter, 0, sizeof(unsigned long long), cs));
                p.row_begin = (int32_t)c0;
                p.row_end = (int32_t)c1;
                const int64_t g = std::min<int64_t>(c.grid, c1 - c0);
                CK(fill2_launch(p, c.nt, h->w, mode, c.vis, (int)g, c.smem, cs));
                h->launches += 1;
            }
            continue;
        }
        const int grid = c.grid < rows ? c.grid : rows;
        CK(fill2_launch(p, c.nt, h->w, mode, c.vis, grid, c.smem, cs));
        h->launches += 1;
    }
    if (forked)  // join
        for (size_t k = 1; k < h->classes.size(); ++k) {
            cudaEvent_t je = set ? h->cls_doneS[set][k] : h->classes[k].done;
            CK(cudaEventRecord(je, set ? h->cls_streamS[set][k] : h->classes[k].stream));
            CK(cudaStreamWaitEvent(s, je, 0));
        }
    return LU_OK;
}

// Extra traversal scratch sets 1..kSets-1 (same sizes as set 0), their class streams and the
// pipeline's streams; allocated on the first pipelined lu_sym_run_host call.
lu_status ensure_sets(lu_sym *h, bool *fits)
{
    *fits = true;
    if (h->dbitmapS[kSets - 1]) return LU_OK;
    int64_t need_spill = 0, need_stg = 0;
    for (auto &c : h->classes) {
        need_spill = std::max<int64_t>(need_spill, c.spill_off + 2 * c.cap * (int64_t)c.grid);
        need_stg = std::max<int64_t>(need_stg, c.stg_off + c.cap * (int64_t)c.grid);
    }
    // the two extra sets must fit the budget too (else lu_sym_run_host runs unpipelined)
    const uint64_t extra = (uint64_t)(kSets - 1) *
                           ((uint64_t)need_spill * 4 + (h->staging ? (uint64_t)need_stg * 4 : 0) +
                            (uint64_t)h->map_words * 4 * (h->gbitmap ? 2 : 1));
    if ((uint64_t)h->scratch_bytes + extra > h->budget) {
        *fits = false;
        return LU_OK;
    }
    lu_status st;
    for (int k = 1; k < kSets; ++k) {
        if ((st = salloc(h, &h->gspillS[k], (size_t)need_spill)) != LU_OK) return st;
        if (h->gbitmap && (st = salloc(h, &h->gbitmapS[k], (size_t)h->map_words)) != LU_OK)
            return st;
        if (h->staging && (st = salloc(h, &h->stgS[k], (size_t)need_stg)) != LU_OK) return st;
        h->cls_streamS[k].assign(h->classes.size(), nullptr);
        h->cls_doneS[k].assign(h->classes.size(), nullptr);
        for (size_t c = 0; c < h->classes.size(); ++c) {
            CK(cudaEventCreateWithFlags(&h->cls_doneS[k][c], cudaEventDisableTiming));
            if (c > 0)
                CK(cudaStreamCreateWithFlags(&h->cls_streamS[k][c], cudaStreamNonBlocking));
        }
        if ((st = salloc(h, &h->dbitmapS[k], (size_t)h->map_words)) != LU_OK) return st;
    }
    int lo = 0, hi = 0;
    CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    // [0], [3] count streams of sets 1 and 2 (normal priority); [1] scan + place and [2]
    // device->host copies at the highest priority, so a chunk's placement CTAs go ahead of
    // queued traversal CTAs
    CK(cudaStreamCreateWithPriority(&h->pipe_stream[0], cudaStreamNonBlocking, lo));
    CK(cudaStreamCreateWithPriority(&h->pipe_stream[3], cudaStreamNonBlocking, lo));
    CK(cudaStreamCreateWithPriority(&h->pipe_stream[1], cudaStreamNonBlocking, hi));
    CK(cudaStreamCreateWithPriority(&h->pipe_stream[2], cudaStreamNonBlocking, hi));
    CK(cudaMallocHost(reinterpret_cast<void **>(&h->pin), 2 * sizeof(int64_t)));
    return LU_OK;
}

// Staging pool (HBM): allocated on the first staged count, kept for the handle's lifetime.
lu_status ensure_pool(lu_sym *h)
{
    if (h->pool || h->pool_cap < 0) return LU_OK;
    size_t free_b = 0, total_b = 0;
    CK(mem_info(&free_b, &total_b));
    uint64_t want = h->opts.pool_bytes;
    if (want == 0) {
        const uint64_t budget = h->budget > (uint64_t)h->scratch_bytes
                                    ? h->budget - (uint64_t)h->scratch_bytes : 0;
        want = budget < (32ull << 30) ? budget : (32ull << 30);
        if (want > (uint64_t)(0.9 * (double)free_b)) want = (uint64_t)(0.9 * (double)free_b);
    }
    int64_t cap = (int64_t)(want / sizeof(int32_t));
    if (cap < 1) {
        h->pool_cap = -1;  // no room: every row is re-traversed by emit
        return LU_OK;
    }
    cudaError_t e = scratch_alloc_raw(h, reinterpret_cast<void **>(&h->pool),
                                      (size_t)cap * sizeof(int32_t));
    if (e != cudaSuccess) {
        cudaGetLastError();
        h->pool = nullptr;
        h->pool_cap = -1;
        return LU_OK;
    }
    h->pool_cap = cap;
    h->scratch_bytes += cap * (int64_t)sizeof(int32_t);
    return LU_OK;
}

// Scratch of the row-merge tail (reading G8), allocated on the first count that may defer
// rows: the deferred / failed row lists and, per tail CTA, a frontier spill (2 x n entries), a
// wait list (defer_max) and, when n/8 bytes do not fit shared memory, an HBM visited slot.
// One 1024-thread CTA per SM, fewer if the scratch budget is short (none: deferral is off).
lu_status ensure_merge(lu_sym *h)
{
    if (h->defer_list || h->defer_win <= 0) return LU_OK;
    int sms = 0, smem_optin = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device));
    CK(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, h->device));
    const int n = h->n;
    // a cluster of G CTAs per deferred row (bitmap sliced over their shared memories), else
    // one CTA with the bitmap in shared memory, else in an HBM slot
    // 8 CTAs: with the first two rows on the whole grid, the tail's critical path is one
    // hub's closure on its cluster (cfg3 tail 14.7 ms with 4, 12.4 with 8, 15.0 with 16;
    // profiles/r02/merge_cluster_size.log)
    int g = 8;
    if (const char *e = getenv("LUSYM_MERGE_CLUSTER")) g = atoi(e);  // A/B knob; 1 = no cluster
    h->merge_mode = -1;
    int max_rows = std::min(sms, h->defer_max);
    if (g > 1 && !getenv("LUSYM_MERGE_HBM_BITMAP")) {
        // with the per-CTA filter of other ranks' bits when it fits (LUSYM_MERGE_NOFILTER: A/B)
        for (int f = getenv("LUSYM_MERGE_NOFILTER") ? 0 : 1; f >= 0 && h->merge_mode < 0; --f) {
            const size_t sm = merge_smem_bytes(n, 2, g, h->merge_q, f != 0);
            int clusters = 0;
            if (sm <= (size_t)smem_optin && merge_configure(sm) == cudaSuccess &&
                merge_max_clusters(g, sm, &clusters) == cudaSuccess && clusters > 0) {
                h->merge_mode = 2;
                h->merge_g = g;
                h->merge_smem = sm;
                h->merge_filter = f ? (int)(((int64_t)n + 31) / 32) : 0;
                max_rows = std::min(clusters, h->defer_max);
            }
            cudaGetLastError();
        }
    }
    if (h->merge_mode < 0) {
        h->merge_g = 1;
        const bool sb = merge_smem_bytes(n, 0, 1, h->merge_q) <= (size_t)smem_optin &&
                        !getenv("LUSYM_MERGE_HBM_BITMAP");  // test knob: the HBM-slot variant
        h->merge_mode = sb ? 0 : 1;
        h->merge_smem = merge_smem_bytes(n, h->merge_mode, 1, h->merge_q);
    }
    h->merge_smem_bm = h->merge_mode != 1;
    if (h->merge_smem > (size_t)smem_optin) {
        h->defer_win = 0;
        return LU_OK;
    }
    const int64_t words = ((int64_t)n + 31) / 32;
    const uint64_t per_cta = (uint64_t)(2 * (int64_t)n + h->defer_max) * 4 +
                             (h->merge_smem_bm ? 0 : (uint64_t)words * 4);
    const uint64_t lists = (uint64_t)2 * h->defer_max * 4;
    const uint64_t left = h->budget > (uint64_t)h->scratch_bytes + lists
                              ? h->budget - (uint64_t)h->scratch_bytes - lists : 0;
    int64_t rows = std::min<int64_t>(max_rows, (int64_t)(left / per_cta) / h->merge_g);
    if (rows < 1) {
        h->defer_win = 0;
        return LU_OK;
    }
    const int64_t grid = rows * h->merge_g;  // CTAs
    CK(merge_configure(h->merge_smem));
    h->merge_grid = (int)grid;
    lu_status st;
    if ((st = salloc(h, &h->defer_list, (size_t)h->defer_max)) != LU_OK) return st;
    if ((st = salloc(h, &h->fail_list, (size_t)h->defer_max)) != LU_OK) return st;
    if ((st = salloc(h, &h->mspill, (size_t)grid * 2 * (size_t)n)) != LU_OK) return st;
    if ((st = salloc(h, &h->mwait, (size_t)grid * (size_t)h->defer_max)) != LU_OK) return st;
    if (!h->merge_smem_bm) {
        if ((st = salloc(h, &h->mgbitmap, (size_t)grid * (size_t)words)) != LU_OK) return st;
        CK(cudaMemsetAsync(h->mgbitmap, 0, (size_t)grid * (size_t)words * 4, h->stream));
    }
    // the grid-wide mode for short lists (k_merge_grid): whole-GPU scratch
    // LUSYM_MERGE_GRID_MAX (A/B knob, off by default): deferred-row lists of at most that many
    // rows are finished by the whole grid, one row at a time (k_merge_grid), instead of by
    // 4-CTA clusters in parallel.  Measured on cfg3's 32 hubs: 19.1 ms against 17.4 (396
    // rounds; the per-round phases and grid barriers cost what the extra SMs save).
    // mg_head > 0: the grid takes only the first rows of a list and the clusters the rest.
    h->mg_max = 0;
    if (const char *e = getenv("LUSYM_MERGE_GRID_MAX")) h->mg_max = atoi(e);
    // LUSYM_MERGE_GRID_HEAD: the grid takes the first rows of every list (default 2): the
    // head of the hubs' chain, whose closure is the cluster tail's critical path (cfg3 tail
    // 16.5 -> 15.2-15.3 ms with 2 or 3, profiles/r02/merge_grid_head.log)
    h->mg_head = 2;
    if (const char *e = getenv("LUSYM_MERGE_GRID_HEAD")) h->mg_head = atoi(e);
    if ((h->mg_max > 0 || h->mg_head > 0) &&
        merge_grid_size(n, &h->mg_grid, &h->mg_filter) == cudaSuccess &&
        h->mg_grid > 0) {
        const size_t need = (size_t)words * 4 + (size_t)2 * n * 4 + (size_t)4 * n * 8 + 64 * 8 +
                            ((size_t)4 * h->mg_grid + 8) * 8 + 64;
        const uint64_t left2 = h->budget > (uint64_t)h->scratch_bytes
                                   ? h->budget - (uint64_t)h->scratch_bytes : 0;
        if (need <= left2) {
            if ((st = salloc(h, &h->mg_bits, (size_t)words)) != LU_OK) return st;
            if ((st = salloc(h, &h->mg_q, (size_t)2 * n)) != LU_OK) return st;
            if ((st = salloc(h, &h->mg_ll, (size_t)4 * n + 64 + 4 * (size_t)h->mg_grid + 8)) !=
                LU_OK)
                return st;
            if ((st = salloc(h, &h->mg_ctrl, 16)) != LU_OK) return st;
            CK(cudaMemsetAsync(h->mg_bits, 0, (size_t)words * 4, h->stream));
        } else {
            h->mg_max = h->mg_head = 0;
        }
    } else {
        cudaGetLastError();
        h->mg_max = h->mg_head = 0;
    }
    return LU_OK;
}

// [0, row_end) covered by the staged ranges (every row a deferred row may need is staged)
bool staged_below(const lu_sym *h, int32_t row_end)
{
    std::vector<std::pair<int32_t, int32_t>> r = h->staged;
    std::sort(r.begin(), r.end());
    int32_t reach = 0;
    for (auto &x : r) {
        if (x.first > reach) break;
        reach = std::max(reach, x.second);
    }
    return reach >= row_end;
}

// The row-merge tail after a pass that deferred rows: sort the deferred list, finish the rows
// by closure over the staged rows (k_merge_rows), then let fill2 finish (stage) whatever the
// tail could not — its list length is read on the device, so no host round trip.
// The row-merge tail over `list` (ascending, *list_cnt rows on the device, at most list_max):
// finish the rows by closure over the staged rows (k_merge_rows), then let fill2 finish
// (stage) whatever the tail could not — its list length is read on the device, so no host
// round trip.  wait / fail_list hold list_max entries (per tail CTA / in total).
lu_status run_tail_list(lu_sym *h, int32_t *fill_count, const int32_t *list,
                        unsigned long long *slots, int32_t list_max, int32_t *wait,
                        int32_t *fail_list, cudaStream_t s)
{
    MergeParams mp;
    mp.n = h->n;
    mp.rp = h->rp;
    mp.ci = h->ci;
    mp.pool = h->pool;
    mp.pool_cap = h->pool_cap;
    mp.pool_cursor = h->dstats + kSlotPoolCursor;
    mp.row_off = h->row_off;
    mp.ucut = h->ucut;
    mp.fill_count = fill_count;
    mp.list = list;
    mp.list_cnt = slots;
    mp.list_max = list_max;
    mp.counter = slots + 1;
    mp.gbitmap = h->mgbitmap;
    mp.gb_stride = ((int64_t)h->n + 31) / 32;
    mp.spill = h->mspill;
    mp.spill_cap = h->n;
    mp.wait = wait;
    mp.fail_list = fail_list;
    mp.fail_cnt = slots + 2;
    mp.stats = slots + 3;
    mp.q = h->merge_q;
    mp.cl_filter = h->merge_mode == 2 ? h->merge_filter : 0;
    if (h->mg_max > 0 || h->mg_head > 0) {
        // a short list: the whole grid, one row at a time (k_merge_grid); a longer one is left
        // to the clusters (the kernel checks the device-side count)
        const size_t n = (size_t)h->n;
        mp.grid_max = h->mg_max;
        mp.grid_head = h->mg_head;
        mp.gbits = h->mg_bits;
        mp.gq = h->mg_q;
        mp.glen = h->mg_ll;
        mp.goff = h->mg_ll + n;
        mp.gcoff = h->mg_ll + 2 * n;
        mp.gstart = h->mg_ll + 3 * n;
        mp.gpart = h->mg_ll + 4 * n + 64;
        mp.gctrl = h->mg_ctrl;
        mp.grid_filter = h->mg_filter;
        if (merge_grid_launch(mp, h->mg_grid, s) == cudaSuccess) {
            h->launches += 1;
        } else {
            // a cooperative launch that cannot be made (e.g. a shared GPU): the clusters, whose
            // claims then start at the first row, take the whole list
            cudaGetLastError();
            h->mg_max = h->mg_head = 0;
        }
    }
    CK(merge_launch(mp, h->merge_mode, h->merge_g, h->merge_grid, h->merge_smem, s));
    h->launches += 2;
    lu_status st = run_pass(h, kStage, 0, h->n, fill_count, nullptr, nullptr, s, fail_list, 0,
                            0, false, slots + 2);
    h->tail_ran = true;
    return st;
}

// The tail after a pass that deferred rows (its own list, sorted first).
lu_status run_tail(lu_sym *h, int32_t *fill_count, cudaStream_t s)
{
    ev_begin(h, kEvTail, s);
    unsigned long long *slots = h->dstats + kSlotDefer;
    CK(merge_sort_list(h->defer_list, slots, h->defer_max, s));
    lu_status st = run_tail_list(h, fill_count, h->defer_list, slots, h->defer_max, h->mwait,
                                 h->fail_list, s);
    ev_end(h, kEvTail, s);
    return st;
}

}  // namespace

extern "C" {

int32_t lu_sym_abi_version(void) { return LU_SYM_ABI_VERSION; }

void lu_sym_default_opts(lu_sym_opts *o)
{
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->struct_size = (int32_t)sizeof(lu_sym_opts);
}

const char *lu_status_str(lu_status s)
{
    switch (s) {
    case LU_OK: return "LU_OK";
    case LU_ERR_ARG: return "LU_ERR_ARG";
    case LU_ERR_INPUT: return "LU_ERR_INPUT";
    case LU_ERR_NOMEM: return "LU_ERR_NOMEM";
    case LU_ERR_CAPACITY: return "LU_ERR_CAPACITY";
    case LU_ERR_CUDA: return "LU_ERR_CUDA";
    case LU_ERR_STATE: return "LU_ERR_STATE";
    case LU_ERR_INTERNAL: return "LU_ERR_INTERNAL";
    }
    return "LU_ERR_UNKNOWN";
}

const char *lu_last_error(void) { return g_err.c_str(); }

lu_status lu_sym_create(lu_sym **out, int32_t n, int64_t nnz_a, const int64_t *d_row_ptr,
                        const int32_t *d_col_idx, const lu_sym_opts *opts, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_create"};
    g_err.clear();
    if (!out) return fail(LU_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (n < 0 || nnz_a < 0) return fail(LU_ERR_ARG, "negative size (n=%d, nnz=%lld)", n,
                                         (long long)nnz_a);
    if (!d_row_ptr || (nnz_a > 0 && !d_col_idx)) return fail(LU_ERR_ARG, "null CSR pointer");
    if (opts && opts->struct_size != (int32_t)sizeof(lu_sym_opts))
        return fail(LU_ERR_ARG, "opts.struct_size %d != %zu", opts->struct_size,
                    sizeof(lu_sym_opts));
    cudaStream_t s = (cudaStream_t)stream;
    lu_sym *h = new lu_sym();
    h->stream = s;
    if (opts) h->opts = *opts; else lu_sym_default_opts(&h->opts);
    memset(&h->stats, 0, sizeof(h->stats));
    h->n = n;
    h->nnz_a = nnz_a;
    h->rp = d_row_ptr;
    h->ci = d_col_idx;
    cudaEvent_t t0, t1;
    lu_status st = LU_OK;
    auto bail = [&](lu_status e) {
        free_handle(h);
        return e;
    };
    if (cudaGetDevice(&h->device) != cudaSuccess) return bail(fail(LU_ERR_CUDA, "no device"));
    if (cudaEventCreate(&t0) != cudaSuccess || cudaEventCreate(&t1) != cudaSuccess)
        return bail(fail(LU_ERR_CUDA, "cudaEventCreate failed"));
    cudaEventRecord(t0, s);
    g_tc = std::chrono::steady_clock::now();
    auto lap = [&](const char *what) { dbg_lap(s, what); };
    if ((st = dalloc(h, &h->dstats, kStatSlots)) != LU_OK) return bail(st);
    if ((st = dalloc(h, &h->dbad, 2)) != LU_OK) return bail(st);
    if ((st = dalloc(h, &h->scan_blk, scan_scratch_elems(n))) != LU_OK) return bail(st);
    cudaMemsetAsync(h->dstats, 0, kStatSlots * sizeof(unsigned long long), s);
    // S1: validate A
    {
        cudaError_t e = validate_csr(n, nnz_a, d_row_ptr, d_col_idx, h->dbad, s);
        unsigned long long bad = ~0ull;
        if (e == cudaSuccess) e = cudaMemcpyAsync(&bad, h->dbad, 8, cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e != cudaSuccess)
            return bail(fail(LU_ERR_CUDA, "validate: %s", cudaGetErrorString(e)));
        if (bad != ~0ull) {
            static const char *what[] = {"", "row_ptr[0] != 0", "row_ptr not monotone",
                                         "row_ptr[n] != nnz", "column index out of [0,n)",
                                         "row not strictly increasing (unsorted or duplicate)"};
            const int code = (int)(bad & 0xff);
            return bail(fail(LU_ERR_INPUT, "invalid CSR at row %lld: %s",
                             (long long)(bad >> 8), what[code < 6 ? code : 0]));
        }
    }
    lap("validate");
    if (n == 0) {
        cudaEventDestroy(t0);
        cudaEventDestroy(t1);
        *out = h;
        return LU_OK;
    }
    // traversal adjacency slots W: the smallest of 4 / 6 / 8 that holds nearly every vertex's
    // off-diagonal entries (rows are stored 4 or 8 wide; larger rows are heavy records)
    {
        int w = h->opts.ell_width;
        if (w != 0 && w != 4 && w != 6 && w != 8)
            return bail(fail(LU_ERR_ARG, "ell_width must be 0, 4, 6 or 8 (got %d)", w));
        for (int cand = 4; w == 0 && cand <= 8; cand += 2) {
            unsigned long long light = 0;
            cudaError_t e = count_light(n, d_row_ptr, d_col_idx, cand, h->dstats + 15, s);
            if (e == cudaSuccess)
                e = cudaMemcpyAsync(&light, h->dstats + 15, 8, cudaMemcpyDeviceToHost, s);
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
            if (e != cudaSuccess) return bail(fail(LU_ERR_CUDA, "%s", cudaGetErrorString(e)));
            if (cand == 8 || light >= (unsigned long long)(0.995 * n)) w = cand;
        }
        h->w = w;
        lap("ell width");
        if ((st = dalloc(h, &h->ell, (size_t)n * (w <= 4 ? 4 : 8))) != LU_OK) return bail(st);
        cudaError_t e = build_ell(n, d_row_ptr, d_col_idx, w, h->ell, s);
        if (e != cudaSuccess) return bail(fail(LU_ERR_CUDA, "%s", cudaGetErrorString(e)));
        {  // rows scanned by a whole warp from A's CSR (off-diagonal degree > W)
            unsigned long long light = 0;
            e = count_light(n, d_row_ptr, d_col_idx, w, h->dstats + 15, s);
            if (e == cudaSuccess)
                e = cudaMemcpyAsync(&light, h->dstats + 15, 8, cudaMemcpyDeviceToHost, s);
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
            if (e != cudaSuccess) return bail(fail(LU_ERR_CUDA, "%s", cudaGetErrorString(e)));
            h->stats.heavy_rows = n - (int64_t)light;
        }
        // the encoded copy read by the shared-map kernels' BFS (only n whose bitmap can fit
        // shared memory can have such classes)
        if (n <= (1 << 21)) {
            if ((st = dalloc(h, &h->elle, (size_t)n * (w <= 4 ? 4 : 8))) != LU_OK) return bail(st);
            e = encode_ell(n, w, LUSYM_SWZ != 0, h->ell, h->elle, s);
            if (e != cudaSuccess) return bail(fail(LU_ERR_CUDA, "%s", cudaGetErrorString(e)));
        }
    }
    lap("ell build");
    if ((st = plan(h)) != LU_OK) return bail(st);
    lap("plan");
    cudaEventRecord(t1, s);
    if (cudaEventSynchronize(t1) != cudaSuccess)
        return bail(fail(LU_ERR_CUDA, "create: %s", cudaGetErrorString(cudaGetLastError())));
    float ms = 0;
    cudaEventElapsedTime(&ms, t0, t1);
    cudaEventDestroy(t0);
    cudaEventDestroy(t1);
    h->stats.ms_create = ms;
    *out = h;
    return LU_OK;
}

lu_status lu_sym_count(lu_sym *h, int32_t row_begin, int32_t row_end, int32_t *d_fill_count,
                       void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_count"};
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    if (row_begin < 0 || row_end > h->n || row_begin > row_end)
        return fail(LU_ERR_ARG, "row range [%d,%d) outside [0,%d]", row_begin, row_end, h->n);
    if (row_begin == row_end) return LU_OK;
    if (!d_fill_count) return fail(LU_ERR_ARG, "d_fill_count is NULL");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    h->stream = s;
    ev_begin(h, kEvCount, s);
    int mode = kCount;
    bool defer = false, global_defer = false;
    h->tail_ran = false;
    h->deferred_pending = false;
    // LU_F_COUNT_TE: a statistics handle, counts only (the edge counting is compiled into the
    // count kernels alone, so the staged pass carries no per-vertex test for it)
    if (h->staging && !(h->opts.flags & LU_F_COUNT_TE)) {
        if ((st = ensure_merge(h)) != LU_OK) return st;
        st = ensure_pool(h);
        if (st != LU_OK) return st;
        if (h->pool) {
            mode = kStage;
            bool overlap = false;
            for (auto &r : h->staged)
                if (row_begin < r.second && r.first < row_end) overlap = true;
            if (overlap || h->staged.empty()) {  // restart the pool
                h->staged.clear();
                CK(cudaMemsetAsync(h->row_off, 0xff, sizeof(int64_t) * (size_t)h->n, s));
                CK(cudaMemsetAsync(h->dstats + kSlotPoolCursor, 0, 2 * sizeof(unsigned long long),
                                   s));
            }
            h->staged.emplace_back(row_begin, row_end);
            // deferred rows need every row below them staged (reading G8), or the pattern
            // assembled across GPUs (LU_F_DEFER_GLOBAL: no tail here, lu_sym_merge_deferred)
            // (a row has at most i thresholds, so rows below defer_win cannot be deferred)
            global_defer = (h->opts.flags & LU_F_DEFER_GLOBAL) != 0;
            defer = h->defer_win > 0 && h->defer_list && row_end > h->defer_win &&
                    (global_defer || staged_below(h, row_end));
        }
    }
    if (defer) CK(cudaMemsetAsync(h->dstats + kSlotDefer, 0, 6 * sizeof(unsigned long long), s));
    h->defer_active = defer;
    h->defer_from = row_begin;
    st = run_pass(h, mode, row_begin, row_end, d_fill_count, nullptr, nullptr, s);
    h->defer_active = false;
    if (st == LU_OK && defer && !global_defer) st = run_tail(h, d_fill_count, s);
    if (defer && global_defer) {  // deferred rows keep count 0 until lu_sym_merge_deferred
        h->deferred_pending = true;
        CK(zero_deferred_counts(h->defer_list, h->dstats + kSlotDefer, h->defer_max,
                                d_fill_count, s));
    }
    ev_end(h, kEvCount, s);
    return st;
}

lu_status lu_sym_scan(lu_sym *h, const int32_t *d_fill_count, int64_t *d_row_ptr_lu,
                      int64_t *nnz_lu, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_scan"};
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    if (!d_row_ptr_lu || (h->n > 0 && !d_fill_count))
        return fail(LU_ERR_ARG, "null pointer");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    h->stream = s;
    ev_begin(h, kEvScan, s);
    CK(scan_counts(h->n, d_fill_count, d_row_ptr_lu, h->scan_blk, s));
    h->launches += h->n > 0 ? 3 : 1;
    ev_end(h, kEvScan, s);
    int64_t nnz = 0;
    CK(cudaMemcpyAsync(&nnz, d_row_ptr_lu + h->n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    h->nnz_lu = nnz;
    h->stats.nnz_lu = nnz;
    h->scanned = true;
    if (nnz_lu) *nnz_lu = nnz;
    return LU_OK;
}

lu_status lu_sym_emit(lu_sym *h, int32_t row_begin, int32_t row_end, const int64_t *d_row_ptr_lu,
                      int32_t *d_col_idx_lu, int64_t cap, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_emit"};
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    if (row_begin < 0 || row_end > h->n || row_begin > row_end)
        return fail(LU_ERR_ARG, "row range [%d,%d) outside [0,%d]", row_begin, row_end, h->n);
    if (!h->scanned) return fail(LU_ERR_STATE, "lu_sym_emit before lu_sym_scan");
    if (row_begin == row_end) return LU_OK;
    if (!d_row_ptr_lu || !d_col_idx_lu) return fail(LU_ERR_ARG, "null pointer");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    h->stream = s;
    int64_t need = 0;
    CK(cudaMemcpyAsync(&need, d_row_ptr_lu + row_end, sizeof(int64_t), cudaMemcpyDeviceToHost,
                       s));
    CK(cudaStreamSynchronize(s));
    if (cap < need)
        return fail(LU_ERR_CAPACITY, "cap %lld < %lld entries needed", (long long)cap,
                    (long long)need);
    ev_begin(h, kEvEmit, s);
    int64_t retraverse = row_end - row_begin;
    if (h->staging && !h->staged.empty()) {
        // symbolic_2 for the staged rows: place them; re-traverse only the others
        int64_t first = 0;
        CK(cudaMemcpyAsync(&first, d_row_ptr_lu + row_begin, sizeof(int64_t),
                           cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        CK(place_rows(row_begin, row_end, d_row_ptr_lu, h->row_off, h->pool, d_col_idx_lu, first,
                      need - first, s));
        CK(collect_unstaged(row_begin, row_end, h->row_off, h->unstaged, h->dstats + kSlotList,
                            s));
        unsigned long long nun = 0;
        CK(cudaMemcpyAsync(&nun, h->dstats + kSlotList, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        h->launches += 2;
        retraverse = (int64_t)nun;
        if (nun > 0)
            st = run_pass(h, kEmit, row_begin, row_end, nullptr, d_row_ptr_lu, d_col_idx_lu, s,
                          h->unstaged, (int32_t)nun);
    } else {
        st = run_pass(h, kEmit, row_begin, row_end, nullptr, d_row_ptr_lu, d_col_idx_lu, s);
    }
    ev_end(h, kEvEmit, s);
    if (st != LU_OK) return st;
    h->stats.rows_retraversed = retraverse;
    unsigned long long err = 0;
    CK(cudaMemcpyAsync(&err, h->dstats + 5 + kStatErr, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (err)
        return fail(LU_ERR_INTERNAL, "%llu rows emitted a length different from their count",
                    err);
    return LU_OK;
}

lu_status lu_sym_run(lu_sym *h, int32_t *d_fill_count, int64_t *d_row_ptr_lu,
                     int32_t *d_col_idx_lu, int64_t cap, int64_t *nnz_lu, void *stream)
{
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    if (!d_col_idx_lu) {
        lu_status st = lu_sym_count(h, 0, h->n, d_fill_count, stream);
        if (st != LU_OK) return st;
        return lu_sym_scan(h, d_fill_count, d_row_ptr_lu, nnz_lu, stream);
    }
    if (!h->scanned) return fail(LU_ERR_STATE, "second lu_sym_run call before the first");
    if (nnz_lu) *nnz_lu = h->nnz_lu;
    if (cap < h->nnz_lu)
        return fail(LU_ERR_CAPACITY, "cap %lld < nnz %lld", (long long)cap,
                    (long long)h->nnz_lu);
    return lu_sym_emit(h, 0, h->n, d_row_ptr_lu, d_col_idx_lu, cap, stream);
}

lu_status lu_sym_nnz_bound(lu_sym *h, int64_t *bound, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_nnz_bound"};
    g_err.clear();
    if (!h || !bound) return fail(LU_ERR_ARG, "null pointer");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    h->stream = s;
    CK(nnz_upper_bound(h->n, h->rp, h->ci, bound, s));
    h->launches += h->n > 0 ? 4 : 0;
    return LU_OK;
}

lu_status lu_sym_run_host(lu_sym *h, int32_t nchunks, int32_t *d_fill_count,
                          int64_t *d_row_ptr_lu, int32_t *d_col_idx_lu, int64_t cap,
                          int64_t *h_row_ptr_lu, int32_t *h_col_idx_lu, int64_t *nnz_lu,
                          void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_run_host"};
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    if (nchunks < 0 || nchunks > kMaxChunks)
        return fail(LU_ERR_ARG, "nchunks %d outside [0,%d]", nchunks, (int)kMaxChunks);
    if (cap < 0) return fail(LU_ERR_ARG, "cap < 0");
    if (!d_row_ptr_lu || (h->n > 0 && (!d_fill_count || (cap > 0 && !d_col_idx_lu))))
        return fail(LU_ERR_ARG, "null pointer");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    cudaStream_t s = (cudaStream_t)stream;
    h->stream = s;
    const int32_t n = h->n;
    if (nchunks == 0)  // 16 chunks, but none under 4096 rows (each chunk costs a host sync)
        nchunks = std::max(1, std::min(16, n / 4096));
    if (nchunks > n) nchunks = n > 0 ? n : 1;
    bool sets_fit = true;
    if (h->staging) {
        if ((st = ensure_merge(h)) != LU_OK) return st;
        if (h->opts.pool_bytes == 0 && !h->pool && h->pool_cap >= 0 && nchunks > 1) {
            // leave room for the pipeline's two extra scratch sets before the pool takes the rest
            if ((st = ensure_sets(h, &sets_fit)) != LU_OK) return st;
        }
        if ((st = ensure_pool(h)) != LU_OK) return st;
    }
    if (sets_fit && h->staging && h->pool && n > 0 && nchunks > 1)
        if ((st = ensure_sets(h, &sets_fit)) != LU_OK) return st;
    if (!h->staging || !h->pool || n == 0 || nchunks == 1 || !sets_fit) {
        // one chunk, two-pass mode or no pool: the plain calls, then the copies
        int64_t nnz = 0;
        if ((st = lu_sym_run(h, d_fill_count, d_row_ptr_lu, nullptr, 0, &nnz, stream)) != LU_OK)
            return st;
        if (nnz_lu) *nnz_lu = nnz;
        if (cap < nnz)
            return fail(LU_ERR_CAPACITY, "cap %lld < nnz %lld", (long long)cap, (long long)nnz);
        if (nnz > 0 && (st = lu_sym_run(h, d_fill_count, d_row_ptr_lu, d_col_idx_lu, cap, &nnz,
                                         stream)) != LU_OK)
            return st;
        if (h_row_ptr_lu)
            CK(cudaMemcpyAsync(h_row_ptr_lu, d_row_ptr_lu, sizeof(int64_t) * ((size_t)n + 1),
                               cudaMemcpyDeviceToHost, s));
        if (h_col_idx_lu && nnz > 0)
            CK(cudaMemcpyAsync(h_col_idx_lu, d_col_idx_lu, sizeof(int32_t) * (size_t)nnz,
                               cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        return LU_OK;
    }
    // row chunks of equal a-priori traversal cost (row_ptr[i+1]: the TE bound of row i, exact on
    // the grids); offsets are chained in increasing row order
    if ((int)h->chunk_bounds.size() != nchunks + 1) {
        std::vector<int64_t> rp((size_t)n + 1);
        CK(cudaMemcpyAsync(rp.data(), h->rp, sizeof(int64_t) * rp.size(), cudaMemcpyDeviceToHost,
                           s));
        CK(cudaStreamSynchronize(s));
        double total = 0;
        for (int32_t i = 0; i < n; ++i) total += (double)rp[(size_t)i + 1] + 1.0;
        h->chunk_bounds.assign(1, 0);
        double acc = 0;
        for (int32_t i = 0; i < n && (int)h->chunk_bounds.size() < nchunks; ++i) {
            acc += (double)rp[(size_t)i + 1] + 1.0;
            if (acc >= total * (double)h->chunk_bounds.size() / nchunks &&
                i + 1 > h->chunk_bounds.back())
                h->chunk_bounds.push_back(i + 1);
        }
        while ((int)h->chunk_bounds.size() < nchunks + 1) h->chunk_bounds.push_back(n);
        h->chunk_bounds.back() = n;
        // rows of very high degree (circuit hubs, ordered last) make the last chunk's rows the
        // critical path: start that chunk first (a-priori test: max degree > 64 x mean)
        int64_t maxdeg = 0;
        for (int32_t i = 0; i < n; ++i)
            maxdeg = std::max<int64_t>(maxdeg, rp[(size_t)i + 1] - rp[(size_t)i]);
        h->heavy_last = (double)maxdeg > 64.0 * ((double)rp[(size_t)n] / n + 1.0);
    }
    const std::vector<int32_t> &b = h->chunk_bounds;
    for (auto &row : h->pipe_ev)  // events of chunks 0..nchunks-1 and the fork slot
        for (int k = 0; k <= kMaxChunks; ++k)
            if (!row[k] && (k < nchunks || k == kMaxChunks))
                CK(cudaEventCreateWithFlags(&row[k], cudaEventDisableTiming));
    cudaStream_t cs[kSets] = {s, h->pipe_stream[0], h->pipe_stream[3]};
    cudaStream_t sp = h->pipe_stream[1], sc = h->pipe_stream[2];
    cudaEvent_t *ev_count = h->pipe_ev[0], *ev_scan = h->pipe_ev[1], *ev_place = h->pipe_ev[2],
                *ev_copy = h->pipe_ev[3];
    ev_begin(h, kEvCount, s);
    // a fresh staging pool, statistics and row_ptr_lu[0] = 0, then fork the pipeline streams
    h->staged.clear();
    h->staged.emplace_back(0, n);
    h->scanned = false;
    CK(cudaMemsetAsync(h->row_off, 0xff, sizeof(int64_t) * (size_t)n, s));
    CK(cudaMemsetAsync(h->dstats + kSlotPoolCursor, 0, 2 * sizeof(unsigned long long), s));
    CK(cudaMemsetAsync(h->dstats + 1, 0, sizeof(unsigned long long) * kStatCount, s));
    CK(cudaMemsetAsync(d_row_ptr_lu, 0, sizeof(int64_t), s));
    // rows of the last chunk may be deferred to the row-merge tail (reading G8): it runs once
    // every chunk is traversed, and only the last chunk's scan waits for it
    const bool defer = h->defer_win > 0 && h->defer_list != nullptr && n > h->defer_win;
    h->tail_ran = false;
    if (defer) CK(cudaMemsetAsync(h->dstats + kSlotDefer, 0, 6 * sizeof(unsigned long long), s));
    CK(cudaEventRecord(ev_count[kMaxChunks], s));
    for (cudaStream_t x : {cs[1], cs[2], sp, sc})
        CK(cudaStreamWaitEvent(x, ev_count[kMaxChunks], 0));
    // symbolic_1 with staging, chunks in increasing order alternating on sets 1 and 2, so chunk
    // k+1's CTAs fill the SMs chunk k leaves as it drains.  With heavy_last, the last chunk
    // (holding the critical-path rows, L272) starts first on set 0.
    const bool hl = h->heavy_last;
    auto set_of = [&](int k) { return hl && k == nchunks - 1 ? 0 : 1 + (k & 1); };
    for (int pos = 0; pos < nchunks; ++pos) {
        const int k = hl ? (pos == 0 ? nchunks - 1 : pos - 1) : pos;
        const int set = set_of(k);
        h->defer_active = defer && k == nchunks - 1;
        h->defer_from = b[k];
        st = b[k] < b[k + 1] ? run_pass(h, kStage, b[k], b[k + 1], d_fill_count, nullptr, nullptr,
                                        cs[set], nullptr, 0, set, false)
                             : LU_OK;
        h->defer_active = false;
        if (st != LU_OK) return st;
        CK(cudaEventRecord(ev_count[k], cs[set]));
    }
    for (int k = nchunks - 1; k >= 0 && k >= nchunks - 3; --k)  // the last chunk of each set
        CK(cudaStreamWaitEvent(s, ev_count[k], 0));
    if (defer) {  // s follows every chunk's traversal: finish the deferred rows
        if ((st = run_tail(h, d_fill_count, s)) != LU_OK) return st;
        CK(cudaEventRecord(ev_count[nchunks - 1], s));
    }
    CK(cudaEventRecord(h->ev[kEvCount][1], s));  // s now follows every chunk's traversal
    h->ev_used[kEvCount] = true;
    // per chunk, behind its traversal: chained prefix sum, placement (symbolic_2 of staged
    // rows) and the device->host copies of its rows
    int64_t base = 0;
    bool overflow = false;
    ev_begin(h, kEvEmit, sp);
    for (int k = 0; k < nchunks; ++k) {
        const int32_t r0 = b[k], r1 = b[k + 1];
        CK(cudaStreamWaitEvent(sp, ev_count[k], 0));
        CK(scan_counts(r1 - r0, d_fill_count + r0, d_row_ptr_lu + r0, h->scan_blk, sp, true));
        h->launches += r1 > r0 ? 3 : 1;
        CK(cudaMemcpyAsync(h->pin, d_row_ptr_lu + r1, sizeof(int64_t), cudaMemcpyDeviceToHost,
                           sp));
        CK(cudaEventRecord(ev_scan[k], sp));
        CK(cudaEventSynchronize(ev_scan[k]));
        const int64_t end = h->pin[0];
        if (end > cap) overflow = true;
        if (!overflow) {
            CK(place_rows(r0, r1, d_row_ptr_lu, h->row_off, h->pool, d_col_idx_lu, base,
                          end - base, sp));
            h->launches += end > base ? 1 : 0;
        }
        CK(cudaEventRecord(ev_place[k], sp));
        CK(cudaStreamWaitEvent(sc, ev_place[k], 0));
        if (h_row_ptr_lu)
            CK(cudaMemcpyAsync(h_row_ptr_lu + r0, d_row_ptr_lu + r0,
                               sizeof(int64_t) * ((size_t)(r1 - r0) + (k == nchunks - 1)),
                               cudaMemcpyDeviceToHost, sc));
        if (h_col_idx_lu && !overflow && end > base)
            CK(cudaMemcpyAsync(h_col_idx_lu + base, d_col_idx_lu + base,
                               sizeof(int32_t) * (size_t)(end - base), cudaMemcpyDeviceToHost, sc));
        CK(cudaEventRecord(ev_copy[k], sc));
        base = end;
    }
    const int64_t nnz = base;
    CK(cudaEventRecord(h->ev[kEvEmit][1], sp));
    h->ev_used[kEvEmit] = true;
    // join everything into the caller's stream
    CK(cudaStreamWaitEvent(s, ev_place[nchunks - 1], 0));
    CK(cudaStreamWaitEvent(s, ev_copy[nchunks - 1], 0));
    h->nnz_lu = nnz;
    h->stats.nnz_lu = nnz;
    h->scanned = true;
    if (nnz_lu) *nnz_lu = nnz;
    if (overflow) {
        CK(cudaStreamSynchronize(s));
        return fail(LU_ERR_CAPACITY, "cap %lld < nnz %lld", (long long)cap, (long long)nnz);
    }
    // rows that did not fit the staging pool: symbolic_2 by traversal, then copy everything
    CK(collect_unstaged(0, n, h->row_off, h->unstaged, h->dstats + kSlotList, s));
    unsigned long long nun = 0;
    CK(cudaMemcpyAsync(&nun, h->dstats + kSlotList, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    h->launches += 1;
    h->stats.rows_retraversed = (int64_t)nun;
    if (nun > 0) {
        if ((st = run_pass(h, kEmit, 0, n, nullptr, d_row_ptr_lu, d_col_idx_lu, s, h->unstaged,
                           (int32_t)nun)) != LU_OK)
            return st;
        if (h_col_idx_lu && nnz > 0)
            CK(cudaMemcpyAsync(h_col_idx_lu, d_col_idx_lu, sizeof(int32_t) * (size_t)nnz,
                               cudaMemcpyDeviceToHost, s));
        unsigned long long err = 0;
        CK(cudaMemcpyAsync(&err, h->dstats + 5 + kStatErr, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (err)
            return fail(LU_ERR_INTERNAL, "%llu rows emitted a length different from their count",
                        err);
    }
    return LU_OK;
}

lu_status lu_levelize(lu_sym *h, int32_t n, const int64_t *d_row_ptr_lu,
                      const int32_t *d_col_idx_lu, int32_t dep_rule, int32_t *d_level,
                      int32_t *num_levels, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_levelize"};
    g_err.clear();
    if (n < 0) return fail(LU_ERR_ARG, "n < 0");
    if (dep_rule != LU_DEP_U && dep_rule != LU_DEP_GLU3)
        return fail(LU_ERR_ARG, "dep_rule %d", dep_rule);
    if (n > 0 && (!d_row_ptr_lu || !d_col_idx_lu || !d_level))
        return fail(LU_ERR_ARG, "null pointer");
    if (h) {
        lu_status st = check_device(h);
        if (st != LU_OK) return st;
    }
    cudaStream_t s = (cudaStream_t)stream;
    if (h) h->stream = s;
    LevelizeScratch tmp;
    LevelizeScratch &scr = h ? h->lev : tmp;
    const int flags = h ? h->opts.flags : 0;
    const char *where = "";
    LevelizeInfo info;
    if (h) ev_begin(h, kEvLev, s);
    cudaError_t e = levelize_run(n, d_row_ptr_lu, d_col_idx_lu, dep_rule,
                                 !(flags & LU_F_NO_PRUNE), !(flags & LU_F_NO_CONTRACT),
                                 (flags & LU_F_KAHN_WIDE_ONLY) != 0, scr, d_level, &info, s,
                                 &where);
    if (h) ev_end(h, kEvLev, s);
    if (!h) levelize_free(tmp, s);
    if (e != cudaSuccess)
        return fail(e == cudaErrorMemoryAllocation ? LU_ERR_NOMEM : LU_ERR_CUDA,
                    "levelize: %s: %s", where, cudaGetErrorString(e));
    if (num_levels) *num_levels = info.num_levels;
    if (h) {
        h->launches += info.launches;
        h->stats.num_levels = info.num_levels;
        h->stats.levelize_wide_levels = info.wide_rounds;
        h->stats.levelize_narrow_levels = info.narrow_rounds;
        h->stats.levelize_rank_rounds = info.rank_rounds;
    }
    return LU_OK;
}

lu_status lu_level_schedule(int32_t n, const int32_t *d_level, int32_t num_levels,
                            int64_t *d_level_ptr, int32_t *d_level_cols, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_level_schedule"};
    g_err.clear();
    if (n < 0 || num_levels < 0) return fail(LU_ERR_ARG, "negative size");
    if (!d_level_ptr || (n > 0 && (!d_level || !d_level_cols)))
        return fail(LU_ERR_ARG, "null pointer");
    if (n > 0 && num_levels < 1) return fail(LU_ERR_ARG, "num_levels must be >= 1 when n > 0");
    cudaStream_t s = (cudaStream_t)stream;
    int bad = 0;
    CK(level_schedule(n, d_level, num_levels, d_level_ptr, d_level_cols, &bad, s));
    if (bad) return fail(LU_ERR_ARG, "a level is outside [0, num_levels)");
    CK(cudaStreamSynchronize(s));
    return LU_OK;
}

lu_status lu_level_types(int32_t n, const int64_t *d_row_ptr_lu, const int32_t *d_col_idx_lu,
                         const int32_t *d_level, int32_t num_levels, int32_t min_cols,
                         int32_t max_sub_a, int32_t *d_type, int64_t *d_sub, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_level_types"};
    g_err.clear();
    if (n < 0 || num_levels < 0) return fail(LU_ERR_ARG, "negative size");
    if (n > 0 && num_levels < 1) return fail(LU_ERR_ARG, "num_levels must be >= 1 when n > 0");
    if (num_levels > 0 && (!d_type || !d_row_ptr_lu || (n > 0 && (!d_level || !d_col_idx_lu))))
        return fail(LU_ERR_ARG, "null pointer");
    if (min_cols <= 0) {
        int dev = 0;
        CK(cudaGetDevice(&dev));
        CK(cudaDeviceGetAttribute(&min_cols, cudaDevAttrMultiProcessorCount, dev));
    }
    if (max_sub_a <= 0) max_sub_a = 32;
    cudaStream_t s = (cudaStream_t)stream;
    CK(level_types(n, d_row_ptr_lu, d_col_idx_lu, d_level, num_levels, min_cols, max_sub_a,
                   d_type, d_sub, s));
    CK(cudaStreamSynchronize(s));
    return LU_OK;
}

lu_status lu_numeric_scatter(int32_t n, const int64_t *d_row_ptr_a, const int32_t *d_col_idx_a,
                             const float *d_val_a, const int64_t *d_row_ptr_lu,
                             const int32_t *d_col_idx_lu, int64_t nnz_lu, float *d_val_lu,
                             void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_numeric_scatter"};
    g_err.clear();
    if (n < 0 || nnz_lu < 0) return fail(LU_ERR_ARG, "negative size");
    if (n > 0 && (!d_row_ptr_a || !d_row_ptr_lu || (nnz_lu > 0 && (!d_col_idx_lu || !d_val_lu))))
        return fail(LU_ERR_ARG, "null pointer");
    if (n > 0) {
        int64_t nnz_a = 0, nnz_p = 0;
        CK(cudaMemcpyAsync(&nnz_a, d_row_ptr_a + n, sizeof(int64_t), cudaMemcpyDeviceToHost,
                           (cudaStream_t)stream));
        CK(cudaMemcpyAsync(&nnz_p, d_row_ptr_lu + n, sizeof(int64_t), cudaMemcpyDeviceToHost,
                           (cudaStream_t)stream));
        CK(cudaStreamSynchronize((cudaStream_t)stream));
        if (nnz_a > 0 && (!d_col_idx_a || !d_val_a)) return fail(LU_ERR_ARG, "null pointer (A)");
        if (nnz_p != nnz_lu) return fail(LU_ERR_ARG, "nnz_lu %lld != row_ptr_lu[n] %lld",
                                          (long long)nnz_lu, (long long)nnz_p);
    }
    int err = 0;
    CK(numeric_scatter(n, d_row_ptr_a, d_col_idx_a, d_val_a, d_row_ptr_lu, d_col_idx_lu, nnz_lu,
                       d_val_lu, &err, (cudaStream_t)stream));
    if (err) return fail(LU_ERR_INPUT, "an entry of A is not in the L+U pattern");
    return LU_OK;
}

lu_status lu_numeric_factor(int32_t n, const int64_t *d_row_ptr_lu, const int32_t *d_col_idx_lu,
                            const int64_t *d_level_ptr, const int32_t *d_level_cols,
                            int32_t num_levels, float *d_val_lu, void *stream)
{
    return lu_numeric_factor_ex(n, d_row_ptr_lu, d_col_idx_lu, d_level_ptr, d_level_cols,
                                num_levels, LU_NUMERIC_SPARSE, d_val_lu, stream);
}

lu_status lu_numeric_factor_ex(int32_t n, const int64_t *d_row_ptr_lu,
                               const int32_t *d_col_idx_lu, const int64_t *d_level_ptr,
                               const int32_t *d_level_cols, int32_t num_levels, int32_t mode,
                               float *d_val_lu, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_numeric_factor_ex"};
    g_err.clear();
    if (mode != LU_NUMERIC_AUTO && mode != LU_NUMERIC_DENSE && mode != LU_NUMERIC_SPARSE)
        return fail(LU_ERR_ARG, "mode %d", mode);
    if (n < 0 || num_levels < 0) return fail(LU_ERR_ARG, "negative size");
    if (n == 0) return LU_OK;
    if (num_levels < 1) return fail(LU_ERR_ARG, "num_levels must be >= 1 when n > 0");
    if (!d_row_ptr_lu || !d_col_idx_lu || !d_level_ptr || !d_level_cols || !d_val_lu)
        return fail(LU_ERR_ARG, "null pointer");
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<int64_t> lp(num_levels + 1);
    CK(cudaMemcpyAsync(lp.data(), d_level_ptr, sizeof(int64_t) * (num_levels + 1),
                       cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (lp[0] != 0 || lp[num_levels] != n) return fail(LU_ERR_ARG, "level_ptr does not cover n");
    for (int32_t l = 0; l < num_levels; ++l)
        if (lp[l + 1] < lp[l]) return fail(LU_ERR_ARG, "level_ptr not monotone");
    {
        // the schedule must be a permutation of the columns under which every GLU3-rule
        // dependency goes to a later level (a U-rule schedule would race; O(nnz) check)
        int bad = 0;
        CK(validate_schedule(n, d_row_ptr_lu, d_col_idx_lu, d_level_ptr, num_levels,
                             d_level_cols, &bad, s));
        if (bad)
            return fail(LU_ERR_ARG, "the level schedule is not a GLU3-rule schedule of this "
                                    "pattern (a column repeated or out of range, or a strict "
                                    "entry (i,j) with level(min(i,j)) >= level(max(i,j)))");
    }
    int dev = 0, sms = 0, bpsm = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    CK(cudaDeviceGetAttribute(&bpsm, cudaDevAttrMaxBlocksPerMultiprocessor, dev));
    // GLU3.0's dense column format needs an n-long map per concurrent CTA: at most
    // M = L / (n sizeof) CTAs (L352).  The paper switches to the sparse format (Alg. 6) when
    // n > L / (TB_max sizeof) (L372), L = device memory (here: free HBM), TB_max = resident CTAs.
    int dense_ctas = 0;
    if (mode != LU_NUMERIC_SPARSE) {
        size_t free_b = 0, total_b = 0;
        CK(cudaMemGetInfo(&free_b, &total_b));
        const double L = 0.5 * (double)free_b;
        const double tb_max = (double)sms * bpsm;
        const bool dense = mode == LU_NUMERIC_DENSE || (double)n <= L / (tb_max * sizeof(float));
        const double m = L / ((double)n * sizeof(int32_t));
        if (dense) dense_ctas = (int)std::max(1.0, std::min(m, (double)sms * 8));
    }
    int err = 0;
    CK(numeric_factor(n, d_row_ptr_lu, d_col_idx_lu, lp.data(), d_level_ptr, d_level_cols,
                      num_levels, sms,
                      d_val_lu, &err, s, dense_ctas));
    if (err & 1) return fail(LU_ERR_INPUT, "zero pivot");
    if (err) return fail(LU_ERR_INPUT, "update outside the L+U pattern");
    return LU_OK;
}

lu_status lu_sym_deferred_flags(lu_sym *h, int32_t *d_flags, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_deferred_flags"};
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    if (h->n > 0 && !d_flags) return fail(LU_ERR_ARG, "d_flags is NULL");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    if (!h->deferred_pending || !h->defer_list) return LU_OK;
    cudaStream_t s = (cudaStream_t)stream;
    CK(deferred_to_flags(h->defer_list, h->dstats + kSlotDefer, h->defer_max, d_flags, s));
    h->launches += 1;
    return LU_OK;
}

lu_status lu_sym_merge_deferred(lu_sym *h, const int32_t *d_flags, int32_t *d_fill_count,
                                int64_t *d_row_ptr_lu, const int32_t *d_col_idx_lu,
                                int64_t *nnz_lu, void *stream)
{
    nvtx3::scoped_range nvtx_range{"lu_sym_merge_deferred"};
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    const int32_t n = h->n;
    if (n > 0 && (!d_flags || !d_fill_count || !d_row_ptr_lu)) return fail(LU_ERR_ARG, "null pointer");
    lu_status st = check_device(h);
    if (st != LU_OK) return st;
    if (!h->staging) return fail(LU_ERR_STATE, "row merge needs the staging pool (not TWO_PASS)");
    cudaStream_t s = (cudaStream_t)stream;
    h->stream = s;
    if ((st = ensure_merge(h)) != LU_OK) return st;
    if ((st = ensure_pool(h)) != LU_OK) return st;
    if (!h->pool || !h->defer_list) return fail(LU_ERR_NOMEM, "no staging pool / tail scratch");
    ev_begin(h, kEvTail, s);
    int64_t nnz0 = 0;
    CK(cudaMemcpyAsync(&nnz0, d_row_ptr_lu + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    int64_t *pos = nullptr;
    int32_t *list = nullptr, *fails = nullptr, *wait = nullptr;
    CK(dev_alloc((void **)&pos, sizeof(int64_t) * ((size_t)n + 1), s));
    // flagged rows in ascending order: an exclusive prefix sum of the flags, then a scatter
    CK(scan_counts(n, d_flags, pos, h->scan_blk, s));
    int64_t nflag = 0;
    CK(cudaMemcpyAsync(&nflag, pos + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (nnz0 > 0 && !d_col_idx_lu) {
        dev_free(pos, s);
        return fail(LU_ERR_ARG, "d_col_idx_lu is NULL");
    }
    if ((double)nnz0 + (double)nflag * n > (double)h->pool_cap) {
        dev_free(pos, s);
        return fail(LU_ERR_NOMEM, "staging pool (%lld entries) < assembled pattern %lld + %lld "
                    "deferred rows x n", (long long)h->pool_cap, (long long)nnz0,
                    (long long)nflag);
    }
    const size_t lm = (size_t)std::max<int64_t>(nflag, 1);
    CK(dev_alloc((void **)&list, sizeof(int32_t) * lm, s));
    CK(dev_alloc((void **)&fails, sizeof(int32_t) * lm, s));
    CK(dev_alloc((void **)&wait, sizeof(int32_t) * lm * (size_t)h->merge_grid, s));
    // the assembled pattern becomes the pool: row t at its CSR offset, deferred rows appended
    if (nnz0 > 0)
        CK(cudaMemcpyAsync(h->pool, d_col_idx_lu, sizeof(int32_t) * (size_t)nnz0,
                           cudaMemcpyDeviceToDevice, s));
    CK(prep_merge(n, d_flags, d_row_ptr_lu, d_col_idx_lu, h->row_off, h->ucut, pos, list, s));
    unsigned long long init[6] = {(unsigned long long)nflag, 0, 0, 0, 0, 0};
    unsigned long long *slots = h->dstats + kSlotDefer;
    CK(cudaMemcpyAsync(slots, init, sizeof(init), cudaMemcpyHostToDevice, s));
    unsigned long long cursor = (unsigned long long)nnz0;
    CK(cudaMemcpyAsync(h->dstats + kSlotPoolCursor, &cursor, sizeof(cursor),
                       cudaMemcpyHostToDevice, s));
    CK(cudaMemsetAsync(h->dstats + kSlotUnstaged, 0, sizeof(unsigned long long), s));
    h->launches += 2;
    if (nflag > 0)
        st = run_tail_list(h, d_fill_count, list, slots, (int32_t)nflag, wait, fails, s);
    if (st == LU_OK) {
        CK(scan_counts(n, d_fill_count, d_row_ptr_lu, h->scan_blk, s));
        h->launches += 3;
        int64_t nnz = 0;
        CK(cudaMemcpyAsync(&nnz, d_row_ptr_lu + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        h->nnz_lu = nnz;
        h->stats.nnz_lu = nnz;
        h->scanned = true;
        h->staged.assign(1, std::make_pair(0, n));  // the pool holds every row now
        h->deferred_pending = false;
        if (nnz_lu) *nnz_lu = nnz;
    }
    ev_end(h, kEvTail, s);
    for (void *b : {(void *)pos, (void *)list, (void *)fails, (void *)wait}) dev_free(b, s);
    return st;
}

lu_status lu_sym_get_stats(const lu_sym *hc, lu_sym_stats *out)
{
    g_err.clear();
    if (!hc || !out) return fail(LU_ERR_ARG, "null pointer");
    lu_sym *h = const_cast<lu_sym *>(hc);
    double *ms[kEvN] = {&h->stats.ms_count, &h->stats.ms_scan, &h->stats.ms_emit,
                        &h->stats.ms_levelize, &h->stats.ms_tail};
    for (int k = 0; k < kEvN; ++k) {
        if (!h->ev_used[k]) continue;
        if (cudaEventSynchronize(h->ev[k][1]) != cudaSuccess) continue;
        float v = 0;
        if (cudaEventElapsedTime(&v, h->ev[k][0], h->ev[k][1]) == cudaSuccess) *ms[k] = v;
    }
    if (h->dstats && h->n > 0) {
        unsigned long long st[16] = {};
        if (cudaMemcpy(st, h->dstats, sizeof(st), cudaMemcpyDeviceToHost) == cudaSuccess) {
            h->stats.edges_read_count = (int64_t)st[1 + kStatEdges];
            h->stats.vertices_scanned_count = (int64_t)st[1 + kStatVerts];
            h->stats.edges_read_emit = (int64_t)st[5 + kStatEdges];
            h->stats.vertices_scanned_emit = (int64_t)st[5 + kStatVerts];
            h->stats.spills = (int64_t)(st[1 + kStatSpills] + st[5 + kStatSpills]);
        }
        unsigned long long dt[6] = {};
        if (h->tail_ran && cudaMemcpy(dt, h->dstats + kSlotDefer, sizeof(dt),
                                      cudaMemcpyDeviceToHost) == cudaSuccess) {
            h->stats.rows_deferred = (int64_t)std::min<unsigned long long>(dt[0], h->defer_max);
            h->stats.rows_merge_failed = (int64_t)dt[2];
            h->stats.merge_entries_read = (int64_t)dt[3];
            h->stats.merge_rounds = (int64_t)dt[4];
            h->stats.merge_waits = (int64_t)dt[5];
        } else {
            h->stats.merge_rounds = h->stats.merge_waits = 0;
            h->stats.rows_deferred = h->stats.rows_merge_failed = 0;
            h->stats.merge_entries_read = 0;
            h->stats.ms_tail = 0;
        }
    }
    h->stats.scratch_bytes = h->scratch_bytes;
    h->stats.rows_in_flight = h->grid;
    h->stats.threads_per_row = h->nt > 1024 ? 1024 : h->nt;
    h->stats.smem_bytes_per_row = (int32_t)h->smem;
    h->stats.visited_in_smem = h->gb ? 0 : (h->vis == kVisSmem ? 1 : 2);
    h->stats.row_classes = (int32_t)h->classes.size();
    h->stats.ell_width = h->w;
    h->stats.queue_capacity = h->q;
    h->stats.kernel_launches = h->launches;
    h->stats.pool_bytes = h->pool ? h->pool_cap * (int64_t)sizeof(int32_t) : 0;
    h->stats.sample_mean_sv = h->sparse_sv;
    *out = h->stats;
    return LU_OK;
}

lu_status lu_sym_set_row_profile(lu_sym *h, int64_t *d_prof)
{
    g_err.clear();
    if (!h) return fail(LU_ERR_ARG, "handle is NULL");
    h->row_prof = d_prof;
    return LU_OK;
}

void lu_sym_destroy(lu_sym *h)
{
    if (!h) return;
    free_handle(h);  // stream-ordered frees on the handle's last stream
}

}  // extern "C"
