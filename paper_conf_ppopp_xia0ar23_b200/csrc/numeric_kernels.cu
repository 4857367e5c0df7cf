// Numeric factorization on the symbolic pattern: Algorithm 2 of PAPER.md, the
// hybrid column-based right-looking LU (L165-204), scheduled level by level (L206-208) on the
// level-grouped column schedule (lu_level_schedule, Fig. 1(d)).  float values (the paper's
// precision, L487), no pivoting (reading R29).
//
// Layout: As lives in the CSR of L+U that lu_sym_emit writes (rows sorted, reading R9) — the
// paper's numeric phase reads a sorted CSC with a binary search for As(i,k) (Alg. 6);
// here the search runs over the sorted ROW i for column k, the same search on the transposed
// storage, so the symbolic output is consumed without a transpose of its values.  The only
// derived structure is the column view of strict L (lines 2-6 and 9-11 walk "As(k,j) != 0 for
// k > j"): per column j the rows i and CSR positions of its strict-lower entries, built with a
// counting pass, a CUB scan and an atomic scatter (order inside a column is free: the updates
// of one column commute).
//
// Levels in order (L206-208), by default all in ONE cooperative launch with a grid barrier
// between levels (k_update_levels_coop; one launch per level, k_update_level, is the fallback).
// GLU3.0 picks one of three kernel modes per level type (L208: block per column, warp per
// sub-column, kernel per column); here one kernel covers all three: the level's (sub-column,
// L entry) pairs are flattened over the grid, so a narrow level (type C, often a single column
// on a chain of levels) spreads its pairs over the whole GPU and a wide one (type A) gets one
// pass.  Each pair locates As(i,k) from As(i,j)'s position (rank of k among row i's entries
// past j, Alg. 6's binary search over the rest) and subtracts with a float atomic: columns of
// one level may update the same As(i,k) (a sub-column shared by independent columns).  The
// GLU3 dependency rule (reading R12, LU_DEP_GLU3) guarantees that nothing a level reads — its
// own L columns, its U rows — is written within that level.  The update uses the column's
// undivided entries (reading
// R31), As(i,k) -= As(i,j) * (As(j,k) / As(j,j)), and lines 2-6 (As(k,j) /= As(j,j)) run once
// for all columns at the end: a column's strict-L entries are read only by its own update and
// are final once its level starts, so no barrier separates lines 2-6 from lines 7-14.
#include "internal.h"

#include <cooperative_groups.h>
#include <cub/device/device_scan.cuh>

#include <cstdint>
#include <cstdlib>

#include <vector>

namespace lusym {
namespace {

namespace cg = cooperative_groups;

constexpr int kErrPivot = 1, kErrPattern = 2;
constexpr int64_t kTableBudget = 1ll << 30;  // bytes of pair-position table (16 B per pair)

// warp per row i: diagonal position (or -1) and the strict-lower entry count of every column
__global__ void k_diag_lcount(int32_t n, const int64_t *rp, const int32_t *ci, int64_t *dpos,
                              int32_t *lcnt)
{
    const int i = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    const int lane = threadIdx.x & 31;
    if (i >= n) return;
    if (lane == 0) dpos[i] = -1;
    __syncwarp();
    for (int64_t p = rp[i] + lane; p < rp[i + 1]; p += 32) {
        const int c = ci[p];
        if (c < i)
            atomicAdd(&lcnt[c], 1);
        else if (c == i)
            dpos[i] = p;
    }
}

// warp per row i: strict-lower entry (i, c) -> slot of column c (rows i and CSR positions)
__global__ void k_lfill(int32_t n, const int64_t *rp, const int32_t *ci, int64_t *cursor,
                        int32_t *lrow, int64_t *lpos)
{
    const int i = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    const int lane = threadIdx.x & 31;
    if (i >= n) return;
    for (int64_t p = rp[i] + lane; p < rp[i + 1]; p += 32) {
        const int c = ci[p];
        if (c >= i) break;  // rows are sorted: the strict-lower entries come first
        const int64_t e = atomicAdd(reinterpret_cast<unsigned long long *>(cursor + c), 1ull);
        lrow[e] = i;
        lpos[e] = p;
    }
}

// position of column k in the sorted row [lo, hi) of ci, -1 if absent (Alg. 6's binary search,
// L322-348, on the row-sorted storage)
__device__ __forceinline__ int64_t find_col(const int32_t *ci, int64_t lo, int64_t hi, int k)
{
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        const int c = __ldg(ci + mid);
        if (c == k) return mid;
        if (c < k)
            lo = mid + 1;
        else
            hi = mid;
    }
    return -1;
}

// warp per row: As = A's values at their L+U positions, 0 at fill (Alg. 2's input, L175)
__global__ void k_scatter(int32_t n, const int64_t *rpa, const int32_t *cia, const float *va,
                          const int64_t *rp, const int32_t *ci, float *val, int *err)
{
    const int i = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    const int lane = threadIdx.x & 31;
    if (i >= n) return;
    for (int64_t q = rpa[i] + lane; q < rpa[i + 1]; q += 32) {
        const int64_t p = find_col(ci, rp[i], rp[i + 1], cia[q]);
        if (p < 0)
            atomicOr(err, kErrPattern);
        else
            val[p] = va[q];
    }
}

__global__ void k_zero(int64_t m, float *v)
{
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < m;
         p += (int64_t)gridDim.x * blockDim.x)
        v[p] = 0.f;
}

// Alg. 2 pairs of a column: |strict L(:,j)| * |U(j, >j)| rank-1 updates (0 without a diagonal)
__global__ void k_pairs(int32_t n, const int32_t *cols, const int64_t *rp, const int64_t *dpos,
                        const int64_t *cptr, int64_t *cost)
{
    const int pos = blockIdx.x * blockDim.x + threadIdx.x;
    if (pos > n) return;
    if (pos == n) {
        cost[n] = 0;
        return;
    }
    const int j = cols[pos];
    const int64_t dp = dpos[j];
    cost[pos] = dp < 0 ? 0 : (cptr[j + 1] - cptr[j]) * (rp[j + 1] - dp - 1);
}

// One level of Algorithm 2 (lines 7-14), its (sub-column, L entry) pairs flattened over the
// grid: pair g of the level belongs to the column at position pos of level_cols with
// W[pos] <= g < W[pos+1] (W = exclusive scan of the per-column pair counts in schedule order).
// The update uses the column's undivided entries, As(i,k) -= As(i,j) * (As(j,k) / As(j,j)),
// so it needs no barrier after lines 2-6, which k_divide applies at the end (reading R31).
__device__ __forceinline__ void update_pair(
    int64_t g, int32_t pos0, int32_t pos1, const int64_t *__restrict__ W,
    const int32_t *__restrict__ cols, const int64_t *__restrict__ rp,
    const int32_t *__restrict__ ci, const int64_t *__restrict__ dpos,
    const int64_t *__restrict__ cptr, const int32_t *__restrict__ lrow,
    const int64_t *__restrict__ lpos, float *val, int *err)
{
    int lo = pos0, hi = pos1 - 1;  // last pos in [pos0, pos1) with W[pos] <= g
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (__ldg(W + mid) <= g)
            lo = mid;
        else
            hi = mid - 1;
    }
    const int j = __ldg(cols + lo);
    const int64_t r = g - __ldg(W + lo);
    const int64_t e0 = __ldg(cptr + j);
    const int64_t dp = __ldg(dpos + j), u0 = dp + 1, nu = __ldg(rp + j + 1) - u0;
    // L entry outer, sub-column inner: the lanes of a warp share row i and walk U(j,:),
    // so their loads and atomics hit consecutive addresses of row j and row i
    const int64_t e = r / nu, qu = r - e * nu;
    const int k = __ldg(ci + u0 + qu);
    const float d = val[dp];
    const float u = val[u0 + qu] / d;
    const int i = __ldg(lrow + e0 + e);
    const int64_t pij = __ldg(lpos + e0 + e);
    const float l = val[pij];
    // row i's entries above j contain U(j,:) (the pattern is closed under elimination) and
    // start right after As(i,j), so k sits at rank >= qu among them: a direct hit when the
    // two rows agree (a full band), else a binary search of the rest (Alg. 6)
    const int64_t rend = __ldg(rp + i + 1);
    int64_t p = pij + 1 + qu;
    if (p >= rend || __ldg(ci + p) != k) p = p < rend ? find_col(ci, p, rend, k) : -1;
    if (p < 0) {
        atomicOr(err, kErrPattern);
        return;
    }
    atomicAdd(val + p, -l * u);
}

__global__ void __launch_bounds__(256) k_update_level(
    int32_t pos0, int32_t pos1, int64_t total, const int64_t *__restrict__ W,
    const int32_t *__restrict__ cols, const int64_t *__restrict__ rp,
    const int32_t *__restrict__ ci, const int64_t *__restrict__ dpos,
    const int64_t *__restrict__ cptr, const int32_t *__restrict__ lrow,
    const int64_t *__restrict__ lpos, float *val, int *err)
{
    const int64_t wbase = W[pos0];
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total;
         t += (int64_t)gridDim.x * blockDim.x)
        update_pair(wbase + t, pos0, pos1, W, cols, rp, ci, dpos, cptr, lrow, lpos, val, err);
}

// Positions one pair touches, from the read-only index arrays only (row j's U entry q, the
// pivot dp, As(i,j) at pij, the target As(i,k) at p, -1 if outside the pattern).  The values
// are read after the level barrier; the indices can be resolved before it.
struct PairPos {
    int64_t q, dp, pij, p;
};

__device__ __forceinline__ PairPos pair_pos(
    int64_t g, int32_t pos0, int32_t pos1, const int64_t *__restrict__ W,
    const int32_t *__restrict__ cols, const int64_t *__restrict__ rp,
    const int32_t *__restrict__ ci, const int64_t *__restrict__ dpos,
    const int64_t *__restrict__ cptr, const int32_t *__restrict__ lrow,
    const int64_t *__restrict__ lpos)
{
    int lo = pos0, hi = pos1 - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (__ldg(W + mid) <= g)
            lo = mid;
        else
            hi = mid - 1;
    }
    const int j = __ldg(cols + lo);
    const int64_t r = g - __ldg(W + lo);
    const int64_t e0 = __ldg(cptr + j);
    PairPos pp;
    pp.dp = __ldg(dpos + j);
    const int64_t u0 = pp.dp + 1, nu = __ldg(rp + j + 1) - u0;
    const int64_t e = r / nu, qu = r - e * nu;
    pp.q = u0 + qu;
    const int k = __ldg(ci + pp.q);
    const int i = __ldg(lrow + e0 + e);
    pp.pij = __ldg(lpos + e0 + e);
    const int64_t rend = __ldg(rp + i + 1);
    int64_t p = pp.pij + 1 + qu;
    if (p >= rend || __ldg(ci + p) != k) p = p < rend ? find_col(ci, p, rend, k) : -1;
    pp.p = p;
    return pp;
}

__device__ __forceinline__ void pair_apply(const PairPos &pp, float *val, int *err)
{
    if (pp.p < 0) {
        atomicOr(err, kErrPattern);
        return;
    }
    const float u = val[pp.q] / val[pp.dp];
    atomicAdd(val + pp.p, -val[pp.pij] * u);
}

// All levels in one cooperative launch (persistent grid, kCoopNT threads x co-resident CTAs):
// a grid-wide barrier separates consecutive levels instead of a kernel boundary, which on a
// chain of single-column levels (natural-order grids) is most of the per-level cost.  Each
// thread resolves the positions of its first pair of the NEXT level before the barrier (index
// arrays are read-only), so after it only the three value loads and the atomic remain on the
// chain.
// With TAB, the positions of every pair come from a table built beforehand by one parallel
// pass (k_pair_table, when it fits the budget): one coalesced 16-byte load per pair instead of
// the dependent index chain.
constexpr int kCoopNT = 1024;  // one CTA per SM: 64 registers, no spills
// Non-empty levels in order, built on the host from the pair offsets: one 32-byte record per
// level, so finding the next level is one load instead of lptr -> W.
struct LevelDesc {
    int32_t p0, p1;
    int64_t wb, tot;
    int64_t pad;
};
static_assert(sizeof(LevelDesc) == 32, "LevelDesc is two 16-byte loads");

template <bool TAB>
__global__ void __launch_bounds__(kCoopNT, 1) k_update_levels_coop(
    int32_t num_levels, const LevelDesc *__restrict__ ld, const int64_t *__restrict__ W,
    const int32_t *__restrict__ cols, const int64_t *__restrict__ rp,
    const int32_t *__restrict__ ci, const int64_t *__restrict__ dpos,
    const int64_t *__restrict__ cptr, const int32_t *__restrict__ lrow,
    const int64_t *__restrict__ lpos, const int4 *__restrict__ tab, float *val, int *err)
{
    cg::grid_group grid = cg::this_grid();
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    // level l of the non-empty ones: (pos0, pos1, wbase, total); l = num_levels if none
    auto next_level = [&](int32_t l, int32_t &p0, int32_t &p1, int64_t &wb, int64_t &tot) {
        if (l < num_levels) {
            const int4 a = __ldg(reinterpret_cast<const int4 *>(ld + l));
            const longlong2 b = __ldg(reinterpret_cast<const longlong2 *>(ld + l) + 1);
            p0 = a.x;
            p1 = a.y;
            wb = (int64_t)(uint32_t)a.z | ((int64_t)a.w << 32);
            tot = b.x;
        }
        return l;
    };
    int32_t p0 = 0, p1 = 0;
    int64_t wb = 0, tot = 0;
    auto get = [&](int64_t g) -> PairPos {
        if constexpr (TAB) {
            const int4 v = __ldg(tab + g);
            return PairPos{v.x, v.y, v.z, v.w};
        } else {
            return pair_pos(g, p0, p1, W, cols, rp, ci, dpos, cptr, lrow, lpos);
        }
    };
    int32_t l = next_level(0, p0, p1, wb, tot);
    PairPos pre{};
    if (l < num_levels && tid < tot) pre = get(wb + tid);
    while (l < num_levels) {
        if (tid < tot) pair_apply(pre, val, err);
        for (int64_t t = tid + stride; t < tot; t += stride) pair_apply(get(wb + t), val, err);
        l = next_level(l + 1, p0, p1, wb, tot);
        if (l < num_levels && tid < tot) pre = get(wb + tid);
        grid.sync();
    }
}

// The pair-position table: entry g = positions of pair g (global pair ids, W over all of
// level_cols), int32 fields (callers check nnz(L+U) < 2^31).
__global__ void k_pair_table(int64_t total, int32_t n, const int64_t *__restrict__ W,
                             const int32_t *__restrict__ cols, const int64_t *__restrict__ rp,
                             const int32_t *__restrict__ ci, const int64_t *__restrict__ dpos,
                             const int64_t *__restrict__ cptr, const int32_t *__restrict__ lrow,
                             const int64_t *__restrict__ lpos, int4 *tab)
{
    for (int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; g < total;
         g += (int64_t)gridDim.x * blockDim.x) {
        const PairPos pp = pair_pos(g, 0, n, W, cols, rp, ci, dpos, cptr, lrow, lpos);
        tab[g] = make_int4((int)pp.q, (int)pp.dp, (int)pp.pij, (int)pp.p);
    }
}

// GLU3.0's dense column format (reading R33): the target row i of an update
// is expanded into a dense n-long map of its positions (D[k] = position of As(i,k)), so each
// As(i,k) is addressed directly instead of searched (Alg. 6).  One (column j, L entry (i,j))
// item per CTA at a time; the map is an n-int slot per CTA, which is what caps the concurrent
// CTAs at M = L / (n * sizeof) (L352) — the memory limit the sparse mode removes.
__global__ void __launch_bounds__(256) k_update_level_dense(
    int32_t pos0, int32_t pos1, int64_t total, const int64_t *__restrict__ WL,
    const int32_t *__restrict__ cols, const int64_t *__restrict__ rp,
    const int32_t *__restrict__ ci, const int64_t *__restrict__ dpos,
    const int64_t *__restrict__ cptr, const int32_t *__restrict__ lrow,
    const int64_t *__restrict__ lpos, int32_t n, int32_t *dense, float *val, int *err)
{
    int32_t *D = dense + (size_t)blockIdx.x * n;
    const int64_t wbase = WL[pos0];
    for (int64_t t = blockIdx.x; t < total; t += gridDim.x) {
        const int64_t g = wbase + t;
        int lo = pos0, hi = pos1 - 1;  // last pos with WL[pos] <= g
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (__ldg(WL + mid) <= g) lo = mid; else hi = mid - 1;
        }
        const int j = __ldg(cols + lo);
        const int64_t e = __ldg(cptr + j) + (g - __ldg(WL + lo));
        const int i = __ldg(lrow + e);
        const int64_t pij = __ldg(lpos + e), iend = __ldg(rp + i + 1);
        const int64_t dp = __ldg(dpos + j), jend = __ldg(rp + j + 1);
        for (int64_t p = pij + 1 + threadIdx.x; p < iend; p += blockDim.x) D[__ldg(ci + p)] = (int32_t)p;
        __syncthreads();
        if (dp >= 0) {
            const float l = val[pij], d = val[dp];
            for (int64_t q = dp + 1 + threadIdx.x; q < jend; q += blockDim.x) {
                const int32_t p = D[__ldg(ci + q)];
                if (p < 0) atomicOr(err, kErrPattern);
                else atomicAdd(val + p, -l * (val[q] / d));
            }
        }
        __syncthreads();
        for (int64_t p = pij + 1 + threadIdx.x; p < iend; p += blockDim.x) D[__ldg(ci + p)] = -1;
        __syncthreads();
    }
}

// strict-L entry counts of the columns in schedule order (for the dense mode's item scan)
__global__ void k_lcount_sched(int32_t n, const int32_t *cols, const int64_t *dpos,
                               const int64_t *cptr, int64_t *cnt)
{
    const int pos = blockIdx.x * blockDim.x + threadIdx.x;
    if (pos > n) return;
    if (pos == n) {
        cnt[n] = 0;
        return;
    }
    const int j = cols[pos];
    cnt[pos] = dpos[j] < 0 ? 0 : cptr[j + 1] - cptr[j];
}

// lines 2-6 for every column at once (each column's strict-L entries and pivot are final once
// its level has run), and the pivot check of every column: warp per row i
__global__ void k_divide(int32_t n, const int64_t *rp, const int32_t *ci, const int64_t *dpos,
                         float *val, int *err)
{
    const int i = (int)((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
    const int lane = threadIdx.x & 31;
    if (i >= n) return;
    if (lane == 0 && (dpos[i] < 0 || val[dpos[i]] == 0.f)) atomicOr(err, kErrPivot);
    for (int64_t p = rp[i] + lane; p < rp[i + 1]; p += 32) {
        const int c = ci[p];
        if (c >= i) break;
        const int64_t dp = dpos[c];
        if (dp >= 0) val[p] = val[p] / val[dp];
    }
}

}  // namespace

cudaError_t numeric_scatter(int32_t n, const int64_t *rpa, const int32_t *cia, const float *va,
                            const int64_t *rp, const int32_t *ci, int64_t nnz_lu, float *val,
                            int *h_err, cudaStream_t s)
{
    *h_err = 0;
    if (n <= 0) return cudaSuccess;
    int *err = nullptr;
    cudaError_t e;
    if ((e = dev_alloc((void **)&err, sizeof(int), s)) != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(err, 0, sizeof(int), s)) != cudaSuccess) goto out;
    if (nnz_lu > 0) k_zero<<<1184, 256, 0, s>>>(nnz_lu, val);
    k_scatter<<<(int)(((int64_t)n * 32 + 255) / 256), 256, 0, s>>>(n, rpa, cia, va, rp, ci, val,
                                                                      err);
    if ((e = cudaGetLastError()) != cudaSuccess) goto out;
    if ((e = cudaMemcpyAsync(h_err, err, sizeof(int), cudaMemcpyDeviceToHost, s)) != cudaSuccess)
        goto out;
    e = cudaStreamSynchronize(s);
out:
    dev_free(err, s);
    return e;
}

cudaError_t numeric_factor(int32_t n, const int64_t *rp, const int32_t *ci,
                           const int64_t *h_level_ptr, const int64_t *level_ptr_d,
                           const int32_t *level_cols,
                           int32_t num_levels, int32_t num_sms, float *val, int *h_err,
                           cudaStream_t s, int dense_ctas)
{
    *h_err = 0;
    if (n <= 0) return cudaSuccess;
    int64_t *dpos = nullptr, *cptr = nullptr, *cursor = nullptr, *lpos = nullptr, *cost = nullptr,
            *W = nullptr;
    int32_t *lcnt = nullptr, *lrow = nullptr;
    int4 *tab = nullptr;
    LevelDesc *ldesc = nullptr;
    int *err = nullptr;
    void *tmp = nullptr;
    int64_t h_nnz_lu = 0;
    size_t tmp_bytes = 0, tmp2_bytes = 0;
    int64_t nl_total = 0;
    std::vector<int64_t> hW;
    const int wgrid = (int)(((int64_t)n * 32 + 255) / 256);
    cudaError_t e;
#define NK(x)                                                                                  \
    do {                                                                                       \
        if ((e = (x)) != cudaSuccess) goto out;                                                \
    } while (0)
    NK(dev_alloc((void **)&dpos, sizeof(int64_t) * n, s));
    NK(dev_alloc((void **)&cptr, sizeof(int64_t) * (n + 1), s));
    NK(dev_alloc((void **)&cursor, sizeof(int64_t) * (n + 1), s));
    NK(dev_alloc((void **)&cost, sizeof(int64_t) * (n + 1), s));
    NK(dev_alloc((void **)&W, sizeof(int64_t) * (n + 1), s));
    NK(dev_alloc((void **)&lcnt, sizeof(int32_t) * (n + 1), s));
    NK(dev_alloc((void **)&err, sizeof(int), s));
    NK(cudaMemsetAsync(lcnt, 0, sizeof(int32_t) * (n + 1), s));
    NK(cudaMemsetAsync(err, 0, sizeof(int), s));
    // column view of strict L: counts, offsets (CUB scan), atomic scatter
    k_diag_lcount<<<wgrid, 256, 0, s>>>(n, rp, ci, dpos, lcnt);
    NK(cudaGetLastError());
    NK(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, lcnt, cptr, n + 1, s));
    NK(cub::DeviceScan::ExclusiveSum(nullptr, tmp2_bytes, cost, W, n + 1, s));
    NK(dev_alloc(&tmp, tmp_bytes > tmp2_bytes ? tmp_bytes : tmp2_bytes, s));
    NK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, lcnt, cptr, n + 1, s));
    NK(cudaMemcpyAsync(&nl_total, cptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NK(cudaMemcpyAsync(&h_nnz_lu, rp + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    NK(cudaStreamSynchronize(s));
    NK(dev_alloc((void **)&lrow, sizeof(int32_t) * (nl_total ? nl_total : 1), s));
    NK(dev_alloc((void **)&lpos, sizeof(int64_t) * (nl_total ? nl_total : 1), s));
    NK(cudaMemcpyAsync(cursor, cptr, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToDevice, s));
    k_lfill<<<wgrid, 256, 0, s>>>(n, rp, ci, cursor, lrow, lpos);
    // pair counts in schedule order and their scan W: level l owns pairs [W[lp[l]], W[lp[l+1]])
    k_pairs<<<(n + 256) / 256, 256, 0, s>>>(n, level_cols, rp, dpos, cptr, cost);
    NK(cudaGetLastError());
    NK(cub::DeviceScan::ExclusiveSum(tmp, tmp2_bytes, cost, W, n + 1, s));
    hW.resize(n + 1);
    NK(cudaMemcpyAsync(hW.data(), W, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost, s));
    NK(cudaStreamSynchronize(s));
    if (dense_ctas > 0) {
        // dense column format (L350-356): items = the levels' L entries in schedule order,
        // one launch per level, dense_ctas CTAs each with an n-int position map
        int64_t *WL = nullptr, *lc = nullptr;
        int32_t *dense = nullptr;
        std::vector<int64_t> hWL((size_t)n + 1);
        NK(dev_alloc((void **)&WL, sizeof(int64_t) * (n + 1), s));
        NK(dev_alloc((void **)&lc, sizeof(int64_t) * (n + 1), s));
        NK(dev_alloc((void **)&dense, sizeof(int32_t) * (size_t)n * dense_ctas, s));
        NK(cudaMemsetAsync(dense, 0xff, sizeof(int32_t) * (size_t)n * dense_ctas, s));
        k_lcount_sched<<<(n + 256) / 256, 256, 0, s>>>(n, level_cols, dpos, cptr, lc);
        NK(cub::DeviceScan::ExclusiveSum(tmp, tmp2_bytes, lc, WL, n + 1, s));
        NK(cudaMemcpyAsync(hWL.data(), WL, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost, s));
        NK(cudaStreamSynchronize(s));
        for (int32_t l = 0; l < num_levels; ++l) {
            const int32_t p0 = (int32_t)h_level_ptr[l], p1 = (int32_t)h_level_ptr[l + 1];
            const int64_t total = hWL[p1] - hWL[p0];
            if (p1 <= p0 || total <= 0 || hW[p1] == hW[p0]) continue;
            const int grid = (int)(total < dense_ctas ? total : dense_ctas);
            k_update_level_dense<<<grid, 256, 0, s>>>(p0, p1, total, WL, level_cols, rp, ci, dpos,
                                                      cptr, lrow, lpos, n, dense, val, err);
        }
        NK(cudaGetLastError());
        NK(cudaStreamSynchronize(s));
        dev_free(WL, s);
        dev_free(lc, s);
        dev_free(dense, s);
    } else
    // levels in order (L206-208): one cooperative launch with a grid barrier per level, or
    // (LUSYM_NUMERIC_LAUNCH_PER_LEVEL=1, or no co-residency) one launch per level with a grid
    // sized to the level's pairs
    {
        int occ = 0;
        const char *ev = getenv("LUSYM_NUMERIC_LAUNCH_PER_LEVEL");
        const bool per_level = ev && ev[0] == '1';
        // pair table when it fits kTableBudget and the int32 fields (LUSYM_NUMERIC_TABLE=0: off)
        const char *et = getenv("LUSYM_NUMERIC_TABLE");
        const int64_t pairs = hW[n], nnz_lu = h_nnz_lu;
        const char *eb = getenv("LUSYM_NUMERIC_TABLE_GB");  // budget override (A/B)
        const int64_t budget = eb ? (int64_t)(atof(eb) * (1ll << 30)) : kTableBudget;
        const bool use_tab = !per_level && !(et && et[0] == '0') && pairs > 0 &&
                             pairs * (int64_t)sizeof(int4) <= budget && nnz_lu < INT32_MAX;
        const void *kfn = use_tab ? (const void *)k_update_levels_coop<true>
                                  : (const void *)k_update_levels_coop<false>;
        if (!per_level) NK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kfn, kCoopNT, 0));
        if (!per_level && occ > 0) {
            if (use_tab) {
                NK(dev_alloc((void **)&tab, sizeof(int4) * pairs, s));
                k_pair_table<<<num_sms * 8, 256, 0, s>>>(pairs, n, W, level_cols, rp, ci, dpos,
                                                          cptr, lrow, lpos, tab);
                NK(cudaGetLastError());
            }
            std::vector<LevelDesc> hd;
            hd.reserve(num_levels);
            for (int32_t l = 0; l < num_levels; ++l) {
                const int32_t a = (int32_t)h_level_ptr[l], b = (int32_t)h_level_ptr[l + 1];
                if (hW[b] > hW[a]) hd.push_back(LevelDesc{a, b, hW[a], hW[b] - hW[a], 0});
            }
            int32_t nlv = (int32_t)hd.size();
            NK(dev_alloc((void **)&ldesc, sizeof(LevelDesc) * (hd.empty() ? 1 : hd.size()), s));
            if (!hd.empty())
                NK(cudaMemcpyAsync(ldesc, hd.data(), sizeof(LevelDesc) * hd.size(),
                                   cudaMemcpyHostToDevice, s));
            const LevelDesc *ld_c = ldesc;
            const int4 *tab_c = tab;
            void *args[] = {&nlv, &ld_c, &W, &level_cols, &rp, &ci, &dpos, &cptr, &lrow, &lpos,
                            &tab_c, &val, &err};
            NK(cudaLaunchCooperativeKernel(kfn, dim3(num_sms * occ), dim3(kCoopNT), args, 0, s));
        } else {
            for (int32_t l = 0; l < num_levels; ++l) {
                const int32_t p0 = (int32_t)h_level_ptr[l], p1 = (int32_t)h_level_ptr[l + 1];
                const int64_t total = hW[p1] - hW[p0];
                if (p1 <= p0 || total <= 0) continue;
                const int64_t blocks = (total + 255) / 256;
                const int grid =
                    (int)(blocks < (int64_t)num_sms * 8 ? blocks : (int64_t)num_sms * 8);
                k_update_level<<<grid, 256, 0, s>>>(p0, p1, total, W, level_cols, rp, ci, dpos,
                                                    cptr, lrow, lpos, val, err);
            }
        }
    }
    NK(cudaGetLastError());
    k_divide<<<wgrid, 256, 0, s>>>(n, rp, ci, dpos, val, err);
    NK(cudaGetLastError());
    NK(cudaMemcpyAsync(h_err, err, sizeof(int), cudaMemcpyDeviceToHost, s));
    NK(cudaStreamSynchronize(s));
#undef NK
out:
    dev_free(dpos, s);
    dev_free(cptr, s);
    dev_free(cursor, s);
    dev_free(cost, s);
    dev_free(W, s);
    dev_free(lcnt, s);
    dev_free(lrow, s);
    dev_free(lpos, s);
    dev_free(err, s);
    dev_free(tmp, s);
    dev_free(tab, s);
    dev_free(ldesc, s);
    return e;
}

}  // namespace lusym
