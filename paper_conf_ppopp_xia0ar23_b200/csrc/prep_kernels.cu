// Preparation kernels: CSR validation (S1), the ELL-W traversal adjacency, and the int64
// prefix sum of the per-row counts (S4, Alg. 3 line 7 "prefix_sum(fill_count_d)", L262).
#include "internal.h"

#include <climits>

namespace lusym {
namespace {

constexpr unsigned kFull = 0xffffffffu;

// Error codes packed with the row id: (row << 8) | code; the smallest row wins.
enum { kBadRp0 = 1, kBadMono = 2, kBadNnz = 3, kBadCol = 4, kBadOrder = 5 };

__global__ void k_validate(int32_t n, int64_t nnz, const int64_t *rp, const int32_t *ci,
                           unsigned long long *bad)
{
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i > n) return;
    auto report = [&](int64_t row, int code) {
        atomicMin(bad, ((unsigned long long)row << 8) | (unsigned long long)code);
    };
    const int64_t a = rp[i];
    if (i == 0 && a != 0) report(0, kBadRp0);
    if (i == n) {
        if (a != nnz) report(n, kBadNnz);
        return;
    }
    const int64_t b = rp[i + 1];
    if (b < a) {
        report(i, kBadMono);
        return;
    }
    const int64_t lo = a < 0 ? 0 : a, hi = b > nnz ? nnz : b;
    int prev = -1;
    for (int64_t k = lo; k < hi; ++k) {
        const int c = ci[k];
        if (c < 0 || c >= n) {
            report(i, kBadCol);
            return;
        }
        if (c <= prev) {
            report(i, kBadOrder);
            return;
        }
        prev = c;
    }
}

// number of rows whose off-diagonal degree is <= w
__global__ void k_count_light(int32_t n, const int64_t *rp, const int32_t *ci, int w,
                              unsigned long long *cnt)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    bool light = false;
    if (i < n) {
        const int64_t a = rp[i], b = rp[i + 1];
        const int64_t len = b - a;
        // light = in the ELL: the diagonal present and at most w off-diagonal entries
        if (len <= w + 1)
            for (int64_t k = a; k < b; ++k)
                if (ci[k] == i) light = true;
    }
    const unsigned m = __ballot_sync(kFull, light);
    if ((threadIdx.x & 31) == 0 && m) atomicAdd(cnt, (unsigned long long)__popc(m));
}

// ell[i*S .. i*S+S), S = 4 (W = 4) or 8 (W = 6, 8): the off-diagonal neighbours of i padded
// with i itself up to W slots (i is always visited when its row is read, so a padded slot is a
// no-op test), or, for degree > W, the heavy record {kHeavy, len, off_lo, off_hi} pointing at
// A's own row (diagonal included: it is always visited when i is scanned, so it is skipped).
template <int W>
__global__ void k_build_ell(int32_t n, const int64_t *rp, const int32_t *ci, int32_t *ell)
{
    constexpr int S = W <= 4 ? 4 : 8;
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int64_t a = rp[i], b = rp[i + 1];
    const int64_t len = b - a;
    int out[S];
#pragma unroll
    for (int s = 0; s < S; ++s) out[s] = s < W ? i : -1;
    bool heavy = len > W + 1;
    if (!heavy) {
        int m = 0;
        bool diag = false;
        for (int64_t k = a; k < b; ++k) {
            const int c = ci[k];
            if (c == i) {
                diag = true;
                continue;
            }
            if (m == W) {
                heavy = true;
                break;
            }
#pragma unroll
            for (int s = 0; s < W; ++s)
                if (s == m) out[s] = c;
            ++m;
        }
        // a light row always has its diagonal, so its traversed edges are its non-padding
        // slots + 1 (fill2 row_edges); a row without one is read from the CSR instead
        if (!diag) heavy = true;
    }
    if (heavy) {
        out[0] = kHeavy;
        out[1] = (int)len;
        out[2] = (int)(uint32_t)(a & 0xffffffffll);
        out[3] = (int)(a >> 32);
#pragma unroll
        for (int s = 4; s < S; ++s) out[s] = -1;
    }
    int4 *dst = reinterpret_cast<int4 *>(ell + (size_t)i * S);
    dst[0] = make_int4(out[0], out[1], out[2], out[3]);
    if constexpr (S == 8) dst[1] = make_int4(out[4], out[5], out[6], out[7]);
}

// shared-map encoding of the light ELL slots (fill2_impl.cuh enc_slot / dec_slot)
__global__ void k_encode_ell(int64_t total, int stride, bool swz, const int32_t *ell,
                             int32_t *elle)
{
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < total;
         k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t row = k / stride;
        const int32_t head = ell[row * stride];
        const int32_t v = ell[k];
        if (head == kHeavy || v < 0) {
            elle[k] = v;
        } else {
            int w = v >> 5;
            if (swz) w ^= (w >> 5) & 31;
            elle[k] = (w << 7) | (v & 31);
        }
    }
}

// entries (i, j) of rows i < bound with j >= bound: pattern marks a split map sends to HBM
__global__ void k_count_far(int32_t n, const int64_t *rp, const int32_t *ci, int32_t bound,
                            unsigned long long *cnt)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned c = 0;
    if (i < n && i < bound) {
        const int64_t a = rp[i];
        for (int64_t k = rp[i + 1] - 1; k >= a && ci[k] >= bound; --k) ++c;  // rows are sorted
    }
    c = __reduce_add_sync(kFull, c);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(cnt, (unsigned long long)c);
}

// ---------------------------------------------------------------- scan (int32 -> int64)
constexpr int kScanNT = 1024;
constexpr int kScanItems = 4;
constexpr int kScanTile = kScanNT * kScanItems;

__device__ __forceinline__ long long block_scan_ll(long long x, long long *s, long long &total)
{
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const long long y = __shfl_up_sync(kFull, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) s[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        long long v = s[lane];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const long long y = __shfl_up_sync(kFull, v, o);
            if (lane >= o) v += y;
        }
        s[lane] = v;
    }
    __syncthreads();
    total = s[31];
    const long long r = (wid ? s[wid - 1] : 0) + inc - x;
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(kScanNT) k_scan_tiles(int32_t n, const int32_t *cnt,
                                                        int64_t *blk)
{
    __shared__ long long s[32];
    const int64_t base = (int64_t)blockIdx.x * kScanTile + threadIdx.x * kScanItems;
    long long sum = 0;
#pragma unroll
    for (int j = 0; j < kScanItems; ++j)
        if (base + j < n) sum += cnt[base + j];
    long long total;
    block_scan_ll(sum, s, total);
    if (threadIdx.x == 0) blk[blockIdx.x] = total;
}

__global__ void __launch_bounds__(kScanNT) k_scan_blocks(int64_t nb, int64_t *blk,
                                                         int64_t *row_ptr_n,
                                                         const int64_t *carry_in)
{
    __shared__ long long s[32];
    long long carry = carry_in ? *carry_in : 0;  // chained scan: offsets continue from row_ptr[0]
    for (int64_t b0 = 0; b0 < nb; b0 += kScanNT) {
        const int64_t b = b0 + threadIdx.x;
        const long long v = b < nb ? blk[b] : 0;
        long long total;
        const long long ex = block_scan_ll(v, s, total);
        if (b < nb) blk[b] = carry + ex;
        carry += total;
    }
    if (threadIdx.x == 0) *row_ptr_n = carry;
}

__global__ void __launch_bounds__(kScanNT) k_scan_final(int32_t n, const int32_t *cnt,
                                                        const int64_t *blk, int64_t *row_ptr)
{
    __shared__ long long s[32];
    const int64_t base = (int64_t)blockIdx.x * kScanTile + threadIdx.x * kScanItems;
    long long v[kScanItems];
    long long sum = 0;
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        v[j] = base + j < n ? cnt[base + j] : 0;
        sum += v[j];
    }
    long long total;
    long long run = blk[blockIdx.x] + block_scan_ll(sum, s, total);
#pragma unroll
    for (int j = 0; j < kScanItems; ++j) {
        if (base + j < n) row_ptr[base + j] = run;
        run += v[j];
    }
}

}  // namespace

cudaError_t validate_csr(int32_t n, int64_t nnz, const int64_t *rp, const int32_t *ci,
                         int64_t *d_bad, cudaStream_t s)
{
    cudaError_t e = cudaMemsetAsync(d_bad, 0xff, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    const int nt = 256;
    const int grid = (int)(((int64_t)n + 1 + nt - 1) / nt);
    k_validate<<<grid, nt, 0, s>>>(n, nnz, rp, ci, reinterpret_cast<unsigned long long *>(d_bad));
    return cudaGetLastError();
}

cudaError_t count_light(int32_t n, const int64_t *rp, const int32_t *ci, int w,
                        unsigned long long *d_cnt, cudaStream_t s)
{
    cudaError_t e = cudaMemsetAsync(d_cnt, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    if (n == 0) return cudaSuccess;
    k_count_light<<<(n + 255) / 256, 256, 0, s>>>(n, rp, ci, w, d_cnt);
    return cudaGetLastError();
}

cudaError_t build_ell(int32_t n, const int64_t *rp, const int32_t *ci, int w, int32_t *ell,
                      cudaStream_t s)
{
    if (n == 0) return cudaSuccess;
    if (w == 4)
        k_build_ell<4><<<(n + 255) / 256, 256, 0, s>>>(n, rp, ci, ell);
    else if (w == 6)
        k_build_ell<6><<<(n + 255) / 256, 256, 0, s>>>(n, rp, ci, ell);
    else
        k_build_ell<8><<<(n + 255) / 256, 256, 0, s>>>(n, rp, ci, ell);
    return cudaGetLastError();
}

cudaError_t encode_ell(int32_t n, int w, bool swz, const int32_t *ell, int32_t *elle,
                       cudaStream_t s)
{
    const int stride = w <= 4 ? 4 : 8;
    const int64_t total = (int64_t)n * stride;
    if (total == 0) return cudaSuccess;
    const int64_t blocks = (total + 255) / 256;
    k_encode_ell<<<(int)(blocks < 4096 ? blocks : 4096), 256, 0, s>>>(total, stride, swz, ell,
                                                                       elle);
    return cudaGetLastError();
}

cudaError_t count_far_entries(int32_t n, const int64_t *rp, const int32_t *ci, int32_t bound,
                              unsigned long long *d_cnt, cudaStream_t s)
{
    cudaError_t e = cudaMemsetAsync(d_cnt, 0, sizeof(unsigned long long), s);
    const int rows = bound < n ? bound : n;
    if (e != cudaSuccess || rows <= 0) return e;
    k_count_far<<<(rows + 255) / 256, 256, 0, s>>>(n, rp, ci, bound, d_cnt);
    return cudaGetLastError();
}

size_t scan_scratch_elems(int32_t n)
{
    return (size_t)(((int64_t)n + kScanTile - 1) / kScanTile) + 1;
}

cudaError_t scan_counts(int32_t n, const int32_t *counts, int64_t *row_ptr, int64_t *blk,
                        cudaStream_t s, bool chained)
{
    const int64_t nb = ((int64_t)n + kScanTile - 1) / kScanTile;
    if (nb > 0) {
        k_scan_tiles<<<(unsigned)nb, kScanNT, 0, s>>>(n, counts, blk);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    k_scan_blocks<<<1, kScanNT, 0, s>>>(nb, blk, row_ptr + n, chained ? row_ptr : nullptr);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess || nb == 0) return e;
    k_scan_final<<<(unsigned)nb, kScanNT, 0, s>>>(n, counts, blk, row_ptr);
    return cudaGetLastError();
}

}  // namespace lusym
