// A-priori capacity of the L+U pattern from A alone (lu_sym_nnz_bound), so that a caller can
// allocate the output before the traversal and stream it out behind it (lu_sym_run_host).
// Theorem 1: (i,j) is in L+U iff a path i -> j exists in G(A) whose
// intermediate vertices are all < min(i,j).
//   j < i: the path's first vertex v1 is in A(i,:) and is j itself or an intermediate < j, so
//          j >= rowmin(i) = min A(i,:).
//   j > i: the path's last intermediate u (if any) is < i and j is in A(u,:), else j is in
//          A(i,:); so j <= max over u <= i of rowmax(u).
// Row i of L+U therefore lies in [min(i, rowmin(i)), max(i, prefix max of rowmax up to i)];
// the bound is the sum of those interval lengths (exact for banded matrices whose band fills,
// e.g. the natural-ordered grids).  Not on the hot path: CUB does the prefix max and the sum.
#include "internal.h"

#include <cub/device/device_reduce.cuh>
#include <cub/device/device_scan.cuh>

namespace lusym {
namespace {

__global__ void k_row_ends(int32_t n, const int64_t *rp, const int32_t *ci, int32_t *rmin,
                           int32_t *rmax)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int64_t a = rp[i], b = rp[i + 1];
    int lo = i, hi = i;
    if (b > a) {  // rows are sorted (validated at create)
        lo = min(lo, ci[a]);
        hi = max(hi, ci[b - 1]);
    }
    rmin[i] = lo;
    rmax[i] = hi;
}

__global__ void k_row_span(int32_t n, const int32_t *rmin, const int32_t *pmax, int64_t *span)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) span[i] = (int64_t)pmax[i] - (int64_t)rmin[i] + 1;
}

struct MaxOp {
    __device__ __forceinline__ int32_t operator()(int32_t a, int32_t b) const
    {
        return a > b ? a : b;
    }
};

}  // namespace

cudaError_t nnz_upper_bound(int32_t n, const int64_t *rp, const int32_t *ci, int64_t *h_bound,
                            cudaStream_t s)
{
    *h_bound = 0;
    if (n <= 0) return cudaSuccess;
    int32_t *rmin = nullptr, *rmax = nullptr, *pmax = nullptr;
    int64_t *span = nullptr, *sum = nullptr;
    void *tmp = nullptr;
    size_t t1 = 0, t2 = 0;
    cudaError_t e = cub::DeviceScan::InclusiveScan(nullptr, t1, rmax, pmax, MaxOp(), n, s);
    if (e == cudaSuccess) e = cub::DeviceReduce::Sum(nullptr, t2, span, sum, n, s);
    const size_t tb = t1 > t2 ? t1 : t2;
    if (e == cudaSuccess) e = dev_alloc((void **)&rmin, sizeof(int32_t) * (size_t)n, s);
    if (e == cudaSuccess) e = dev_alloc((void **)&rmax, sizeof(int32_t) * (size_t)n, s);
    if (e == cudaSuccess) e = dev_alloc((void **)&pmax, sizeof(int32_t) * (size_t)n, s);
    if (e == cudaSuccess) e = dev_alloc((void **)&span, sizeof(int64_t) * (size_t)n, s);
    if (e == cudaSuccess) e = dev_alloc((void **)&sum, sizeof(int64_t), s);
    if (e == cudaSuccess) e = dev_alloc(&tmp, tb ? tb : 1, s);
    if (e == cudaSuccess) {
        k_row_ends<<<(n + 255) / 256, 256, 0, s>>>(n, rp, ci, rmin, rmax);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cub::DeviceScan::InclusiveScan(tmp, t1, rmax, pmax, MaxOp(), n, s);
    if (e == cudaSuccess) {
        k_row_span<<<(n + 255) / 256, 256, 0, s>>>(n, rmin, pmax, span);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cub::DeviceReduce::Sum(tmp, t2, span, sum, n, s);
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(h_bound, sum, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    for (void *p : {(void *)rmin, (void *)rmax, (void *)pmax, (void *)span, (void *)sum, tmp})
        if (p) dev_free(p, s);
    return e;
}

}  // namespace lusym
