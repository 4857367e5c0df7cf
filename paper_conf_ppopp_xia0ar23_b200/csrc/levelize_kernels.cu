// Levelization (S8 + S9): Algorithm 5 of PAPER.md (L290-320) on sm_100a.
//
//   cons_graph   (L308): the dependency graph is a VIEW of the L+U CSR: the successors of
//                column i are the strict-U entries of row i (rule "U(i,j)!=0 => j depends on
//                i", L167), optionally pruned to the prefix up to the first symmetric pair
//                p_i = min{k > i : (i,k),(k,i) in P}, which is exact for longest paths
//                (reading R27); the GLU3 reading (R12) adds the transpose of strict L.
//   cnt_indegree (L311): atomic histogram over the successor lists.
//   Topo         (L293-306): ONE persistent cooperative kernel replaces the parent kernel and
//                its dynamically launched children (device-side cudaDeviceSynchronize is gone
//                on sm_90+).  Wide levels: every CTA relaxes the queue (warp per queued column,
//                lanes over its successors), grid barrier per level.  Narrow levels (queue <=
//                narrow_max): CTA 0 alone runs level after level with a shared-memory queue
//                and __syncthreads, while the other CTAs wait at the next grid barrier.
//   level(k) = max(-1, level(preds)) + 1 (L283) is exactly the round in which column k's
//   in-degree reaches zero; each column is enqueued once, on that decrement (reading R14).
#include "internal.h"

#include <cooperative_groups.h>

namespace cg = cooperative_groups;

namespace lusym {
namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kKahnNT = 512;
constexpr int kNarrowQ = 4096;   // shared queue entries per buffer (narrow phase)
constexpr int kNarrowMax = 2048; // queue size at or below which CTA 0 runs alone

// ctrl block layout (int32)
enum { kQ0 = 0, kQ1 = 1, kQ2 = 2, kLevel = 3, kWide = 4, kNarrow = 5, kCtrlInts = 8 };

__device__ __forceinline__ int64_t lower_bound_dev(const int32_t *ci, int64_t lo, int64_t hi,
                                                   int key)
{
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (ci[mid] < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// One warp per row: strict-U start and (pruned) successor end.
__global__ void k_urange(int32_t n, const int64_t *rp, const int32_t *ci, int prune,
                         int64_t *ustart, int64_t *uend)
{
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = wg; r < n; r += nwarps) {
        const int i = (int)r;
        const int64_t a = rp[i], b = rp[i + 1];
        int64_t us = 0;
        if (lane == 0) us = lower_bound_dev(ci, a, b, i + 1);
        us = __shfl_sync(kFull, us, 0);
        int64_t ue = b;
        if (prune) {
            for (int64_t c0 = us; c0 < b; c0 += 32) {
                const int64_t k = c0 + lane;
                bool hit = false;
                if (k < b) {
                    const int r2 = ci[k];  // (i, r2) in P, r2 > i: is (r2, i) in P too?
                    const int64_t lo = rp[r2], hi = rp[r2 + 1];
                    const int64_t pos = lower_bound_dev(ci, lo, hi, i);
                    hit = pos < hi && ci[pos] == i;
                }
                const unsigned bal = __ballot_sync(kFull, hit);
                if (bal) {
                    ue = c0 + (__ffs(bal) - 1) + 1;
                    break;
                }
            }
        }
        if (lane == 0) {
            ustart[i] = us;
            uend[i] = ue;
        }
    }
}

// GLU3 reading: count strict-L entries per column (transpose sizes).
__global__ void k_lt_count(int32_t n, const int64_t *rp, const int32_t *ci,
                           const int64_t *ustart, int32_t *cnt)
{
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = wg; r < n; r += nwarps) {
        const int64_t a = rp[r], b = ustart[r];
        for (int64_t k = a + lane; k < b; k += 32) {
            const int c = ci[k];
            if (c < r) atomicAdd(cnt + c, 1);
        }
    }
}

__global__ void k_lt_fill(int32_t n, const int64_t *rp, const int32_t *ci, const int64_t *ustart,
                          unsigned long long *cursor, int32_t *lt_idx)
{
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = wg; r < n; r += nwarps) {
        const int64_t a = rp[r], b = ustart[r];
        for (int64_t k = a + lane; k < b; k += 32) {
            const int c = ci[k];
            if (c < r) lt_idx[atomicAdd(cursor + c, 1ull)] = (int)r;
        }
    }
}

// cnt_indegree (L311)
__global__ void k_indeg(int32_t n, const int32_t *ci, const int64_t *us, const int64_t *ue,
                        const int64_t *ltp, const int32_t *lti, int32_t *indeg)
{
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = wg; r < n; r += nwarps) {
        for (int64_t k = us[r] + lane; k < ue[r]; k += 32) atomicAdd(indeg + ci[k], 1);
        if (ltp)
            for (int64_t k = ltp[r] + lane; k < ltp[r + 1]; k += 32) atomicAdd(indeg + lti[k], 1);
    }
}

// cons_queue for level 0 (L294-296)
__global__ void k_init_queue(int32_t n, const int32_t *indeg, int32_t *level, int32_t *q0,
                             int32_t *ctrl)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    const bool src = j < n && indeg[j] == 0;
    if (j < n) level[j] = src ? 0 : -1;
    const unsigned b = __ballot_sync(kFull, src);
    if (!b) return;
    const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(ctrl + kQ0, __popc(b));
    base = __shfl_sync(kFull, base, leader);
    if (src) q0[base + __popc(b & ((1u << lane) - 1u))] = j;
}

struct KahnArgs {
    int32_t n;
    const int32_t *ci;
    const int64_t *us, *ue;
    const int64_t *ltp;
    const int32_t *lti;
    int32_t *indeg, *level, *queue;  // queue: 2 x n
    int32_t *ctrl;
    int32_t narrow_max;
    int32_t wide_only;
};

__device__ __forceinline__ int ld_ctrl(const int32_t *p) { return __ldcg(p); }

// relax every successor v of u: update (L299) + cons_queue (L302) fused
template <class Push>
__device__ __forceinline__ void relax(const KahnArgs &A, int u, int nextlvl, Push &&push)
{
    const int lane = threadIdx.x & 31;
    const int64_t a = A.us[u], b = A.ue[u];
    for (int64_t eb = a; eb < b; eb += 32) {
        const int64_t e = eb + lane;
        bool z = false;
        int v = 0;
        if (e < b) {
            v = A.ci[e];
            z = atomicSub(A.indeg + v, 1) == 1;
            if (z) A.level[v] = nextlvl;
        }
        push(z, v);
    }
    if (A.ltp) {
        const int64_t c = A.ltp[u], d = A.ltp[u + 1];
        for (int64_t eb = c; eb < d; eb += 32) {
            const int64_t e = eb + lane;
            bool z = false;
            int v = 0;
            if (e < d) {
                v = A.lti[e];
                z = atomicSub(A.indeg + v, 1) == 1;
                if (z) A.level[v] = nextlvl;
            }
            push(z, v);
        }
    }
}

__device__ __forceinline__ int warp_push_slot(bool pred, int *cnt, unsigned &b)
{
    b = __ballot_sync(kFull, pred);
    if (!b) return 0;
    const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(cnt, __popc(b));
    base = __shfl_sync(kFull, base, leader);
    return base + __popc(b & ((1u << lane) - 1u));
}

__global__ void __launch_bounds__(kKahnNT) k_kahn(const KahnArgs A)
{
    cg::grid_group grid = cg::this_grid();
    __shared__ int32_t sq[2 * kNarrowQ];
    __shared__ int32_t scnt[3];
    const int tid = threadIdx.x, warp = tid >> 5;
    constexpr int NW = kKahnNT / 32;
    const int gwarp = blockIdx.x * NW + warp;
    const int twarps = gridDim.x * NW;
    int L = 0;
    for (;;) {
        const int q = ld_ctrl(A.ctrl + L % 3);
        if (q == 0) break;
        int32_t *Q = A.queue + (size_t)(L & 1) * A.n;
        int32_t *NQ = A.queue + (size_t)((L + 1) & 1) * A.n;
        if (q <= A.narrow_max && !A.wide_only) {
            if (blockIdx.x == 0) {
                // ---- narrow phase: CTA 0 alone, shared queue, __syncthreads per level
                int32_t *cur = sq, *nxt = sq + kNarrowQ;
                for (int k = tid; k < q; k += kKahnNT) cur[k] = Q[k];
                if (tid == 0) scnt[0] = scnt[1] = scnt[2] = 0;
                __syncthreads();
                int qq = q, it = 0, lv = L, nq = 0;
                for (;;) {
                    int *cnt = &scnt[(it + 1) % 3];
                    if (tid == 0) scnt[(it + 2) % 3] = 0;
                    int32_t *gnext = A.queue + (size_t)((lv + 1) & 1) * A.n;
                    for (int k = warp; k < qq; k += NW) {
                        const int u = cur[k];
                        relax(A, u, lv + 1, [&](bool z, int v) {
                            unsigned b;
                            const int pos = warp_push_slot(z, cnt, b);
                            if (z) {
                                if (pos < kNarrowQ) nxt[pos] = v; else gnext[pos] = v;
                            }
                        });
                    }
                    __syncthreads();
                    nq = *cnt;
                    ++lv;
                    ++it;
                    if (nq == 0 || nq > A.narrow_max) {
                        for (int k = tid; k < nq && k < kNarrowQ; k += kKahnNT) gnext[k] = nxt[k];
                        break;
                    }
                    int32_t *t = cur; cur = nxt; nxt = t;
                    qq = nq;
                    __syncthreads();
                }
                if (tid == 0) {
                    A.ctrl[lv % 3] = nq;
                    A.ctrl[(lv + 1) % 3] = 0;
                    A.ctrl[kLevel] = lv;
                    A.ctrl[kNarrow] += it;
                }
            }
            grid.sync();
            L = ld_ctrl(A.ctrl + kLevel);
            continue;
        }
        // ---- wide level: all CTAs
        if (blockIdx.x == 0 && tid == 0) {
            A.ctrl[(L + 2) % 3] = 0;
            A.ctrl[kWide] += 1;
        }
        int *gcnt = A.ctrl + (L + 1) % 3;
        for (int k = gwarp; k < q; k += twarps) {
            const int u = Q[k];
            relax(A, u, L + 1, [&](bool z, int v) {
                unsigned b;
                const int pos = warp_push_slot(z, gcnt, b);
                if (z) NQ[pos] = v;
            });
        }
        grid.sync();
        ++L;
    }
    if (blockIdx.x == 0 && tid == 0) A.ctrl[kLevel] = L;
}

constexpr int kAuxNT = 256;

int aux_grid(int64_t rows_per_warp_items)
{
    int64_t warps = rows_per_warp_items;
    int64_t blocks = (warps * 32 + kAuxNT - 1) / kAuxNT;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (blocks < 1) blocks = 1;
    return (int)blocks;
}

}  // namespace

void levelize_free(LevelizeScratch &s)
{
    cudaFree(s.ustart); cudaFree(s.uend); cudaFree(s.indeg); cudaFree(s.queue);
    cudaFree(s.lt_ptr); cudaFree(s.lt_idx); cudaFree(s.lt_fill); cudaFree(s.scan_blk);
    cudaFree(s.ctrl);
    s = LevelizeScratch();
}

#define LV_CK(x)                                                                             \
    do {                                                                                     \
        cudaError_t e_ = (x);                                                                \
        if (e_ != cudaSuccess) {                                                             \
            *err = #x;                                                                       \
            return e_;                                                                       \
        }                                                                                    \
    } while (0)

cudaError_t levelize_run(int32_t n, const int64_t *rp_lu, const int32_t *ci_lu, int rule,
                         bool prune, bool wide_only, LevelizeScratch &s, int32_t *level,
                         int32_t *num_levels, int32_t *wide_levels, int32_t *narrow_levels,
                         cudaStream_t st, const char **err)
{
    *num_levels = 0;
    *wide_levels = *narrow_levels = 0;
    if (n == 0) return cudaSuccess;
    if (s.n_cap < n) {
        cudaFree(s.ustart); cudaFree(s.uend); cudaFree(s.indeg); cudaFree(s.queue);
        cudaFree(s.lt_ptr); cudaFree(s.lt_fill); cudaFree(s.scan_blk); cudaFree(s.ctrl);
        s.ustart = s.uend = s.lt_ptr = s.lt_fill = s.scan_blk = nullptr;
        s.indeg = s.queue = s.ctrl = nullptr;
        LV_CK(cudaMalloc(&s.ustart, sizeof(int64_t) * n));
        LV_CK(cudaMalloc(&s.uend, sizeof(int64_t) * n));
        LV_CK(cudaMalloc(&s.indeg, sizeof(int32_t) * n));
        LV_CK(cudaMalloc(&s.queue, sizeof(int32_t) * 2 * (size_t)n));
        LV_CK(cudaMalloc(&s.lt_ptr, sizeof(int64_t) * ((size_t)n + 1)));
        LV_CK(cudaMalloc(&s.lt_fill, sizeof(int64_t) * n));
        LV_CK(cudaMalloc(&s.scan_blk, sizeof(int64_t) * scan_scratch_elems(n)));
        LV_CK(cudaMalloc(&s.ctrl, sizeof(int32_t) * kCtrlInts));
        s.n_cap = n;
    }
    const bool glu3 = rule == 1;
    const int g = aux_grid(n);
    // cons_graph: strict-U ranges (pruned for the U rule)
    k_urange<<<g, kAuxNT, 0, st>>>(n, rp_lu, ci_lu, (prune && !glu3) ? 1 : 0, s.ustart, s.uend);
    LV_CK(cudaGetLastError());
    const int64_t *ltp = nullptr;
    const int32_t *lti = nullptr;
    if (glu3) {
        int32_t *cnt = s.indeg;  // reuse as a temporary int32[n]
        LV_CK(cudaMemsetAsync(cnt, 0, sizeof(int32_t) * n, st));
        k_lt_count<<<g, kAuxNT, 0, st>>>(n, rp_lu, ci_lu, s.ustart, cnt);
        LV_CK(cudaGetLastError());
        LV_CK(scan_counts(n, cnt, s.lt_ptr, s.scan_blk, st));
        int64_t nl = 0;
        LV_CK(cudaMemcpyAsync(&nl, s.lt_ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        LV_CK(cudaStreamSynchronize(st));
        if (s.lt_cap < nl || s.lt_idx == nullptr) {
            cudaFree(s.lt_idx);
            s.lt_idx = nullptr;
            LV_CK(cudaMalloc(&s.lt_idx, sizeof(int32_t) * (size_t)(nl > 0 ? nl : 1)));
            s.lt_cap = nl;
        }
        LV_CK(cudaMemcpyAsync(s.lt_fill, s.lt_ptr, sizeof(int64_t) * n, cudaMemcpyDeviceToDevice,
                              st));
        k_lt_fill<<<g, kAuxNT, 0, st>>>(n, rp_lu, ci_lu, s.ustart,
                                        reinterpret_cast<unsigned long long *>(s.lt_fill),
                                        s.lt_idx);
        LV_CK(cudaGetLastError());
        ltp = s.lt_ptr;
        lti = s.lt_idx;
    }
    // cnt_indegree
    LV_CK(cudaMemsetAsync(s.indeg, 0, sizeof(int32_t) * n, st));
    k_indeg<<<g, kAuxNT, 0, st>>>(n, ci_lu, s.ustart, s.uend, ltp, lti, s.indeg);
    LV_CK(cudaGetLastError());
    // cons_queue (level 0)
    LV_CK(cudaMemsetAsync(s.ctrl, 0, sizeof(int32_t) * kCtrlInts, st));
    k_init_queue<<<(n + 255) / 256, 256, 0, st>>>(n, s.indeg, level, s.queue, s.ctrl);
    LV_CK(cudaGetLastError());
    // Topo: persistent cooperative kernel
    int dev = 0, sms = 0, occ = 0;
    LV_CK(cudaGetDevice(&dev));
    LV_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    LV_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_kahn, kKahnNT, 0));
    if (occ < 1) {
        *err = "k_kahn cannot be resident";
        return cudaErrorLaunchOutOfResources;
    }
    int grid = sms * (occ < 2 ? occ : 2);
    KahnArgs A;
    A.n = n;
    A.ci = ci_lu;
    A.us = s.ustart;
    A.ue = s.uend;
    A.ltp = ltp;
    A.lti = lti;
    A.indeg = s.indeg;
    A.level = level;
    A.queue = s.queue;
    A.ctrl = s.ctrl;
    A.narrow_max = kNarrowMax;
    A.wide_only = wide_only ? 1 : 0;
    void *args[] = {&A};
    LV_CK(cudaLaunchCooperativeKernel((const void *)k_kahn, grid, kKahnNT, args, 0, st));
    int32_t ctrl[kCtrlInts];
    LV_CK(cudaMemcpyAsync(ctrl, s.ctrl, sizeof(ctrl), cudaMemcpyDeviceToHost, st));
    LV_CK(cudaStreamSynchronize(st));
    *num_levels = ctrl[kLevel];
    *wide_levels = ctrl[kWide];
    *narrow_levels = ctrl[kNarrow];
    return cudaSuccess;
}

}  // namespace lusym
