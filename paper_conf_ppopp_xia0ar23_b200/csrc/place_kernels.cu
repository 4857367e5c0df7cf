// symbolic_2 for staged rows (Alg. 3 lines 10-12, "store the locations", L270): the count pass
// (kStage) already wrote every row of L+U, sorted, into an HBM pool at a row-granular offset;
// here the rows are copied to their final CSR slots [rp_lu[i], rp_lu[i+1]).  Output-tiled so
// the copy is load-balanced whatever the row lengths: each CTA owns 4096 consecutive output
// entries, caches the overlapping rows' offsets in shared memory and maps every position to its
// row by binary search.  Rows with row_off < 0 did not fit the pool and are left untouched for
// the traversal fallback.
#include "internal.h"

namespace lusym {
namespace {

constexpr int kPlaceNT = 256;
constexpr int kPlaceTile = 4096;
constexpr int kPlaceRows = 1024;

// Largest r in [lo, hi) with rp[r] <= x, given rp[lo] <= x (rp non-decreasing): a 32-ary
// search by one warp, about log32(rows) dependent loads instead of log2(rows).
__device__ __forceinline__ int warp_row_search(const int64_t *rp, int lo, int hi, int64_t x)
{
    const int lane = threadIdx.x & 31;
    while (hi - lo > 1) {
        const int step = (hi - lo + 31) / 32;
        const int probe = lo + lane * step;
        const bool ok = probe < hi && rp[probe] <= x;
        const unsigned b = __ballot_sync(0xffffffffu, ok);
        const int j = 31 - __clz(b);  // last probe <= x (probe 0 = lo always is)
        lo = lo + j * step;
        hi = min(hi, lo + step);
    }
    return lo;
}

__global__ void __launch_bounds__(kPlaceNT)
    k_place(int32_t rb, int32_t re, const int64_t *rp_lu, const int64_t *row_off,
            const int32_t *pool, int32_t *ci_lu, int64_t base, int64_t total)
{
    __shared__ int64_t srp[kPlaceRows + 1];
    __shared__ int64_t soff[kPlaceRows];
    __shared__ int s_r0, s_nr;
    for (int64_t t0 = (int64_t)blockIdx.x * kPlaceTile; t0 < total;
         t0 += (int64_t)gridDim.x * kPlaceTile) {
        const int64_t s = base + t0;
        const int64_t e = base + (t0 + kPlaceTile < total ? t0 + kPlaceTile : total);
        if (threadIdx.x < 32) {  // rows r0 .. r1 overlap [s, e)
            const int r0 = warp_row_search(rp_lu, rb, re, s);
            const int r1 = warp_row_search(rp_lu, r0, re, e - 1);
            if (threadIdx.x == 0) {
                s_r0 = r0;
                s_nr = r1 - r0 + 1;
            }
        }
        __syncthreads();
        const int r0 = s_r0, nr = s_nr;
        if (nr <= kPlaceRows) {
            for (int k = threadIdx.x; k <= nr; k += kPlaceNT) srp[k] = rp_lu[r0 + k];
            for (int k = threadIdx.x; k < nr; k += kPlaceNT) soff[k] = row_off[r0 + k];
            __syncthreads();
            // kPlaceU positions per thread per round, loads issued before any store
            constexpr int kPlaceU = 4;
            for (int64_t p0 = s + threadIdx.x; p0 < e; p0 += kPlaceNT * kPlaceU) {
                int32_t v[kPlaceU];
                bool ok[kPlaceU];
#pragma unroll
                for (int u = 0; u < kPlaceU; ++u) {
                    const int64_t pos = p0 + (int64_t)u * kPlaceNT;
                    ok[u] = false;
                    v[u] = 0;
                    if (pos < e) {
                        int lo = 0, hi = nr;  // last k with srp[k] <= pos
                        while (hi - lo > 1) {
                            const int mid = (lo + hi) >> 1;
                            if (srp[mid] <= pos) lo = mid; else hi = mid;
                        }
                        const int64_t off = soff[lo];
                        if (off >= 0) {
                            ok[u] = true;
                            v[u] = __ldcs(pool + off + (pos - srp[lo]));
                        }
                    }
                }
#pragma unroll
                for (int u = 0; u < kPlaceU; ++u)
                    if (ok[u]) __stcs(ci_lu + p0 + (int64_t)u * kPlaceNT, v[u]);
            }
        } else {
            for (int64_t pos = s + threadIdx.x; pos < e; pos += kPlaceNT) {
                int lo = r0, hi = r0 + nr;
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (rp_lu[mid] <= pos) lo = mid; else hi = mid;
                }
                const int64_t off = row_off[lo];
                if (off >= 0) ci_lu[pos] = pool[off + (pos - rp_lu[lo])];
            }
        }
        __syncthreads();
    }
}

__global__ void k_collect_unstaged(int32_t rb, int32_t re, const int64_t *row_off,
                                   int32_t *list, unsigned long long *cnt)
{
    const int64_t r = rb + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    // (a row deferred across GPUs, kRowDeferred, is empty until lu_sym_merge_deferred)
    const bool un = r < re && row_off[r] < 0 && row_off[r] != kRowDeferred;
    const unsigned b = __ballot_sync(0xffffffffu, un);
    if (!b) return;
    const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
    unsigned long long base = 0;
    if (lane == leader) base = atomicAdd(cnt, (unsigned long long)__popc(b));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (un) list[base + __popc(b & ((1u << lane) - 1u))] = (int32_t)r;
}

}  // namespace

cudaError_t collect_unstaged(int32_t row_begin, int32_t row_end, const int64_t *row_off,
                             int32_t *list, unsigned long long *cnt, cudaStream_t s)
{
    cudaError_t e = cudaMemsetAsync(cnt, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess || row_end <= row_begin) return e;
    const int nrows = row_end - row_begin;
    k_collect_unstaged<<<(nrows + 255) / 256, 256, 0, s>>>(row_begin, row_end, row_off, list, cnt);
    return cudaGetLastError();
}

cudaError_t place_rows(int32_t row_begin, int32_t row_end, const int64_t *rp_lu,
                       const int64_t *row_off, const int32_t *pool, int32_t *ci_lu,
                       int64_t base, int64_t total, cudaStream_t s)
{
    if (total <= 0) return cudaSuccess;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t tiles = (total + kPlaceTile - 1) / kPlaceTile;
    int64_t cap = (int64_t)sms * 8;
    const int grid = (int)(tiles < cap ? tiles : cap);
    k_place<<<grid, kPlaceNT, 0, s>>>(row_begin, row_end, rp_lu, row_off, pool, ci_lu, base,
                                      total);
    return cudaGetLastError();
}

}  // namespace lusym
