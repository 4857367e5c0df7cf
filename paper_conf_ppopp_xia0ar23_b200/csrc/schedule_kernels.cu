// Level-grouped column schedule: the columns of each level, the form of
// PAPER.md Fig. 1(d) (L72-80, "Column ids for different levels") that the numeric phase's
// level-by-level launches consume (L206-208).  level_ptr[l] .. level_ptr[l+1] delimit the
// columns of level l in level_cols, ascending within a level (reading R15).  Not on the hot
// path: a stable radix sort of (level, column) pairs from CUB does the grouping.  Also the
// GLU3.0 level types A/B/C (L208) that choose the numeric kernel mode per level.
#include "internal.h"

#include <cub/device/device_radix_sort.cuh>

namespace lusym {
namespace {

__global__ void k_iota(int32_t n, int32_t *v)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j < n) v[j] = j;
}

// level_ptr[l] = first position of level l in the sorted keys (keys sorted ascending)
__global__ void k_level_ptr(int32_t n, const int32_t *sorted_level, int32_t num_levels,
                            int64_t *level_ptr)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= n) return;
    const int l = sorted_level[j];
    const int prev = j ? sorted_level[j - 1] : -1;
    for (int k = prev + 1; k <= l; ++k) level_ptr[k] = j;  // levels prev+1..l start here
    if (j == n - 1)
        for (int k = l + 1; k <= num_levels; ++k) level_ptr[k] = n;
}

// GLU3.0 level types (L208): one thread per column j — its sub-columns (reading R28: the
// strict-U entries of row j, As(j,k) != 0 with k > j, Alg. 2 lines 7-14) are the entries of the
// sorted row past the binary-searched position of j; width and sub-columns are accumulated per
// level with integer atomics (exact, order-free).
__global__ void k_level_sub(int32_t n, const int64_t *rp, const int32_t *ci, const int32_t *level,
                            unsigned long long *lsub, unsigned int *lwidth)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= n) return;
    int64_t lo = rp[j], hi = rp[j + 1];
    const int64_t end = hi;
    while (lo < hi) {  // first entry > j
        const int64_t mid = (lo + hi) >> 1;
        if (ci[mid] <= j) lo = mid + 1; else hi = mid;
    }
    const int l = level[j];
    atomicAdd(&lsub[l], (unsigned long long)(end - lo));
    atomicAdd(&lwidth[l], 1u);
}

__global__ void k_level_type(int32_t num_levels, const unsigned long long *lsub,
                             const unsigned int *lwidth, int32_t min_cols, int32_t max_sub_a,
                             int32_t *type, int64_t *sub_out)
{
    const int l = blockIdx.x * blockDim.x + threadIdx.x;
    if (l >= num_levels) return;
    const long long w = lwidth[l], sb = (long long)lsub[l];
    type[l] = w < min_cols ? 2 : (sb <= (long long)max_sub_a * w ? 0 : 1);
    if (sub_out) sub_out[l] = sb;
}

// every level value inside [0, num_levels)
__global__ void k_check_levels(int32_t n, const int32_t *level, int32_t num_levels, int *bad)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j < n && (level[j] < 0 || level[j] >= num_levels)) atomicOr(bad, 1);
}

// schedule -> level of each column; a column listed twice or out of [0, n) is flagged
__global__ void k_sched_levels(int32_t n, const int64_t *level_ptr, int32_t num_levels,
                               const int32_t *cols, int32_t *lvl, int *bad)
{
    const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (q >= n) return;
    int lo = 0, hi = num_levels;  // last l with level_ptr[l] <= q
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (level_ptr[mid] <= q) lo = mid; else hi = mid;
    }
    const int c = cols[q];
    if (c < 0 || c >= n) {
        atomicOr(bad, 1);
        return;
    }
    if (atomicExch(&lvl[c], lo) != -1) atomicOr(bad, 1);
}

// every strict entry (i,j) of L+U makes min(i,j) a GLU3-rule predecessor of max(i,j): its
// level must be lower (one warp per row)
__global__ void k_sched_edges(int32_t n, const int64_t *rp, const int32_t *ci, const int32_t *lvl,
                              int *bad)
{
    const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (w >= n) return;
    const int i = (int)w;
    const int li = lvl[i];
    bool ok = li >= 0;
    for (int64_t p = rp[i] + lane; ok && p < rp[i + 1]; p += 32) {
        const int j = ci[p];
        if (j < 0 || j >= n) { ok = false; break; }
        if (j == i) continue;
        const int lj = lvl[j];
        ok = j < i ? lj < li : li < lj;
    }
    if (!ok) atomicOr(bad, 1);
}

}  // namespace

cudaError_t validate_schedule(int32_t n, const int64_t *rp, const int32_t *ci,
                              const int64_t *level_ptr, int32_t num_levels, const int32_t *cols,
                              int *h_bad, cudaStream_t s)
{
    *h_bad = 0;
    if (n <= 0) return cudaSuccess;
    int32_t *lvl = nullptr;
    int *bad = nullptr;
    cudaError_t e;
    if ((e = dev_alloc((void **)&lvl, sizeof(int32_t) * n, s)) != cudaSuccess) return e;
    if ((e = dev_alloc((void **)&bad, sizeof(int), s)) != cudaSuccess) goto out;
    if ((e = cudaMemsetAsync(lvl, 0xff, sizeof(int32_t) * n, s)) != cudaSuccess) goto out;
    if ((e = cudaMemsetAsync(bad, 0, sizeof(int), s)) != cudaSuccess) goto out;
    k_sched_levels<<<(n + 255) / 256, 256, 0, s>>>(n, level_ptr, num_levels, cols, lvl, bad);
    k_sched_edges<<<(int)(((int64_t)n * 32 + 255) / 256), 256, 0, s>>>(n, rp, ci, lvl, bad);
    if ((e = cudaGetLastError()) != cudaSuccess) goto out;
    if ((e = cudaMemcpyAsync(h_bad, bad, sizeof(int), cudaMemcpyDeviceToHost, s)) != cudaSuccess)
        goto out;
    e = cudaStreamSynchronize(s);
out:
    dev_free(lvl, s);
    dev_free(bad, s);
    return e;
}

cudaError_t level_types(int32_t n, const int64_t *rp, const int32_t *ci, const int32_t *level,
                        int32_t num_levels, int32_t min_cols, int32_t max_sub_a, int32_t *type,
                        int64_t *sub, cudaStream_t s)
{
    if (num_levels <= 0) return cudaSuccess;
    unsigned long long *lsub = nullptr;
    unsigned int *lwidth = nullptr;
    cudaError_t e;
    if ((e = dev_alloc((void **)&lsub, sizeof(unsigned long long) * num_levels, s)) != cudaSuccess)
        return e;
    if ((e = dev_alloc((void **)&lwidth, sizeof(unsigned int) * num_levels, s)) != cudaSuccess)
        goto out;
    if ((e = cudaMemsetAsync(lsub, 0, sizeof(unsigned long long) * num_levels, s)) != cudaSuccess)
        goto out;
    if ((e = cudaMemsetAsync(lwidth, 0, sizeof(unsigned int) * num_levels, s)) != cudaSuccess)
        goto out;
    if (n > 0) k_level_sub<<<(n + 255) / 256, 256, 0, s>>>(n, rp, ci, level, lsub, lwidth);
    k_level_type<<<(num_levels + 255) / 256, 256, 0, s>>>(num_levels, lsub, lwidth, min_cols,
                                                          max_sub_a, type, sub);
    e = cudaGetLastError();
out:
    dev_free(lsub, s);
    dev_free(lwidth, s);
    return e;
}

cudaError_t level_schedule(int32_t n, const int32_t *level, int32_t num_levels,
                           int64_t *level_ptr, int32_t *level_cols, int *h_bad, cudaStream_t s)
{
    *h_bad = 0;
    if (n <= 0) return cudaMemsetAsync(level_ptr, 0, sizeof(int64_t) * (num_levels + 1), s);
    {
        int *bad = nullptr;
        cudaError_t e0 = dev_alloc((void **)&bad, sizeof(int), s);
        if (e0 != cudaSuccess) return e0;
        cudaMemsetAsync(bad, 0, sizeof(int), s);
        k_check_levels<<<(n + 255) / 256, 256, 0, s>>>(n, level, num_levels, bad);
        e0 = cudaMemcpyAsync(h_bad, bad, sizeof(int), cudaMemcpyDeviceToHost, s);
        if (e0 == cudaSuccess) e0 = cudaStreamSynchronize(s);
        dev_free(bad, s);
        if (e0 != cudaSuccess || *h_bad) return e0;
    }
    int32_t *keys_out = nullptr, *vals_in = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    int bits = 1;
    while ((1ll << bits) <= num_levels) ++bits;
    cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, level, keys_out, vals_in,
                                                    level_cols, n, 0, bits, s);
    if (e != cudaSuccess) return e;
    if ((e = dev_alloc((void **)&keys_out, sizeof(int32_t) * n, s)) != cudaSuccess) return e;
    if ((e = dev_alloc((void **)&vals_in, sizeof(int32_t) * n, s)) != cudaSuccess) goto out;
    if ((e = dev_alloc(&tmp, tmp_bytes, s)) != cudaSuccess) goto out;
    k_iota<<<(n + 255) / 256, 256, 0, s>>>(n, vals_in);
    e = cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, level, keys_out, vals_in, level_cols, n, 0,
                                        bits, s);
    if (e != cudaSuccess) goto out;
    k_level_ptr<<<(n + 255) / 256, 256, 0, s>>>(n, keys_out, num_levels, level_ptr);
    e = cudaGetLastError();
out:
    dev_free(keys_out, s);
    dev_free(vals_in, s);
    dev_free(tmp, s);
    return e;
}

}  // namespace lusym
