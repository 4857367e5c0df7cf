// Deferred rows of the count pass, finished by row-merge closure over staged rows (reading G8,
// DESIGN.md §2).
//
// Theorem 1 split at the largest intermediate vertex t of a path i -> j: the
// part i -> t has intermediates < t, the part t -> j too, so for j != i
//     (i,j) in P  iff  A(i,j) != 0  or  (i,t) in P and (t,j) in P for some t < min(i,j).
// Row i of L+U is therefore the least set S with S ⊇ A(i,:) and S ⊇ U_t = {j > t : (t,j) in P}
// for every t in S with t < i (the diagonal comes from A only, reading R7).  A least fixed
// point does not depend on the order its members are expanded in, so one CTA expands a whole
// frontier of new members t < i at once: there is no serial chain of increasing thresholds
// (Alg. 1), which on circuit matrices with hubs ordered last makes a single row cost
// 10^5 dependent threshold windows.  Rows t are read from the staging pool the count pass
// filled (their strict-U part starts ucut[t] entries into the row).
//
// Rows are claimed in increasing order.  A member t that is itself a deferred row still in
// progress is set aside until its CTA publishes it (row_off[t] >= 0, release/acquire); the
// smallest unfinished claimed row never waits, so the resident grid always progresses.  A row
// that cannot be finished (a row it needs is unstaged, or the pool is full) is listed for the
// fill2 fallback launch that follows.
#include "internal.h"

#include <climits>

namespace lusym {
namespace {

constexpr int NT = kMergeNT;
constexpr int NW = NT / 32;
constexpr int kU = 4;  // pool loads in flight per thread

struct MHdr {
    int row, diag, fail, nwait;
    int cnt[2];
    long long off;
    long long red[2][NW];
    long long scan[NW];
};

__device__ __forceinline__ int64_t ld_acquire(const int64_t *p)
{
    int64_t v;
    asm volatile("ld.acquire.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_release(int64_t *p, int64_t v)
{
    asm volatile("st.release.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// exclusive block scan of a 64-bit value; *total = sum over the block
__device__ __forceinline__ long long scan_excl(long long x, MHdr &h, long long *total)
{
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const long long y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) h.scan[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        long long v = lane < NW ? h.scan[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const long long y = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += y;
        }
        if (lane < NW) h.scan[lane] = v;
    }
    __syncthreads();
    *total = h.scan[NW - 1];
    const long long r = (wid ? h.scan[wid - 1] : 0) + inc - x;
    __syncthreads();
    return r;
}

// frontier entry k of buffer b (shared up to q entries, then the CTA's HBM spill half b)
__device__ __forceinline__ int32_t q_get(const int32_t *sq, const int32_t *gq, int q, int64_t k)
{
    return k < q ? sq[k] : __ldcg(gq + k);
}

__device__ __forceinline__ void q_push(bool pred, int32_t w, int *cnt, int32_t *sq, int32_t *gq,
                                       int q)
{
    const unsigned b = __ballot_sync(0xffffffffu, pred);
    if (!b) return;
    const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(cnt, __popc(b));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (pred) {
        const int pos = base + __popc(b & ((1u << lane) - 1u));
        if (pos < q) sq[pos] = w; else gq[pos] = w;
    }
}

// test-and-set of bit v; true iff this call set it
__device__ __forceinline__ bool tas(uint32_t *bm, int v)
{
    const uint32_t b = 1u << (v & 31);
    if (bm[v >> 5] & b) return false;
    return !(atomicOr(bm + (v >> 5), b) & b);
}

template <bool SB>
__global__ void __launch_bounds__(NT, 1) k_merge_rows(const MergeParams p)
{
    extern __shared__ __align__(16) unsigned char smem[];
    MHdr &h = *reinterpret_cast<MHdr *>(smem);
    long long *s_off = reinterpret_cast<long long *>(smem + kHdrBytes);   // [NT]
    long long *s_start = s_off + NT;                                       // [NT]
    int32_t *sq = reinterpret_cast<int32_t *>(s_start + NT);              // 2 x q
    const int nw = (p.n + 31) >> 5;
    uint32_t *bm = SB ? reinterpret_cast<uint32_t *>(sq + 2 * p.q)
                      : p.gbitmap + (size_t)blockIdx.x * p.gb_stride;
    int32_t *gq0 = p.spill + (size_t)blockIdx.x * 2 * p.spill_cap;
    int32_t *wait = p.wait + (size_t)blockIdx.x * p.list_max;
    const int tid = threadIdx.x;
    const int nlist = (int)min(*p.list_cnt, (unsigned long long)p.list_max);
    if (SB)
        for (int w = tid; w < nw; w += NT) bm[w] = 0;
    unsigned long long n_read = 0, n_rounds = 0, n_waits = 0;  // thread 0
    for (;;) {
        if (tid == 0) {
            const unsigned long long c = atomicAdd(p.counter, 1ull);
            h.row = c < (unsigned long long)nlist ? p.list[c] : -1;
            h.diag = 0;
            h.fail = 0;
            h.nwait = 0;
            h.cnt[0] = h.cnt[1] = 0;
        }
        __syncthreads();
        const int i = h.row;
        if (i < 0) break;
        // ---- seed: S = A(i,:); members t < i form the first frontier
        if (tid == 0) atomicOr(bm + (i >> 5), 1u << (i & 31));
        __syncthreads();
        {
            const int64_t rb = p.rp[i], re = p.rp[i + 1];
            for (int64_t b0 = rb; b0 < re; b0 += NT) {
                const int64_t e = b0 + tid;
                int v = -1;
                bool fr = false;
                if (e < re) {
                    v = __ldg(p.ci + e);
                    if (v == i) h.diag = 1;
                    else if (tas(bm, v)) fr = v < i;
                }
                q_push(fr, v, &h.cnt[0], sq, gq0, p.q);
            }
        }
        __syncthreads();
        int cur = 0;
        for (;;) {
            const int fsize = h.cnt[cur];
            if (fsize == 0) {
                const int nwt = h.nwait;
                if (nwt == 0) break;
                // every member left is a deferred row still in progress: wait for them (each
                // was claimed before row i by a running CTA), then expand them
                for (int k = tid; k < nwt; k += NT) {
                    const int t = wait[k];
                    while (ld_acquire(p.row_off + t) == kRowDeferred) __nanosleep(200);
                }
                if (tid == 0) n_waits += nwt;
                __syncthreads();
                for (int k = tid; k < nwt; k += NT) {
                    const int t = wait[k];
                    if (k < p.q) sq[cur * p.q + k] = t; else gq0[(size_t)cur * p.spill_cap + k] = t;
                }
                __syncthreads();
                if (tid == 0) {
                    h.cnt[cur] = nwt;
                    h.nwait = 0;
                }
                __syncthreads();
                continue;
            }
            const int nxt = cur ^ 1;
            const int32_t *fq = sq + cur * p.q, *gfq = gq0 + (size_t)cur * p.spill_cap;
            int32_t *nq = sq + nxt * p.q, *gnq = gq0 + (size_t)nxt * p.spill_cap;
            for (int base = 0; base < fsize; base += NT) {
                const int k = base + tid;
                long long off = 0, len = 0;
                if (k < fsize) {
                    const int t = q_get(fq, gfq, p.q, k);
                    const int64_t o = ld_acquire(p.row_off + t);
                    if (o == kRowDeferred) {
                        wait[atomicAdd(&h.nwait, 1)] = t;
                    } else if (o < 0) {
                        h.fail = 1;  // row t is not in the pool
                    } else {
                        const int uc = __ldcg(p.ucut + t);
                        off = o + uc;
                        len = (long long)__ldcg(p.fill_count + t) - uc;
                    }
                }
                long long total;
                const long long st = scan_excl(len, h, &total);
                s_off[tid] = off;
                s_start[tid] = st;  // non-decreasing; an empty segment shares its successor's start
                __syncthreads();
                if (tid == 0) n_read += (unsigned long long)total;
                // the member owning flat position pos: the last k with s_start[k] <= pos (never an
                // empty segment, and never one past the frontier: those start at total)
                for (long long p0 = 0; p0 < total; p0 += (long long)NT * kU) {
                    int jv[kU];
#pragma unroll
                    for (int u = 0; u < kU; ++u) {
                        const long long pos = p0 + (long long)u * NT + tid;
                        jv[u] = -1;
                        if (pos < total) {
                            int lo = 0;
#pragma unroll
                            for (int step = NT / 2; step >= 1; step >>= 1)
                                if (s_start[lo + step] <= pos) lo += step;
                            jv[u] = __ldcg(p.pool + s_off[lo] + (pos - s_start[lo]));
                        }
                    }
#pragma unroll
                    for (int u = 0; u < kU; ++u) {
                        const int j = jv[u];
                        const bool fr = j >= 0 && tas(bm, j) && j < i;
                        q_push(fr, j, &h.cnt[nxt], nq, gnq, p.q);
                    }
                }
                __syncthreads();
            }
            if (tid == 0) {
                h.cnt[cur] = 0;
                ++n_rounds;
            }
            __syncthreads();
            if (h.fail) break;
            cur = nxt;
        }
        // ---- output: the set bits, ascending, into the pool; publish the row
        if (!h.fail) {
            if (tid == 0 && !h.diag) atomicAnd(bm + (i >> 5), ~(1u << (i & 31)));
            __syncthreads();
            long long c = 0, lo = 0;
            for (int w = tid; w < nw; w += NT) {
                const uint32_t x = bm[w];
                const int pc = __popc(x);
                c += pc;
                if (w < (i >> 5)) lo += pc;
                else if (w == (i >> 5)) lo += __popc(x & ((i & 31) == 31 ? 0xffffffffu
                                                                           : ((2u << (i & 31)) - 1u)));
            }
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                c += __shfl_xor_sync(0xffffffffu, c, o);
                lo += __shfl_xor_sync(0xffffffffu, lo, o);
            }
            if ((tid & 31) == 0) {
                h.red[0][tid >> 5] = c;
                h.red[1][tid >> 5] = lo;
            }
            __syncthreads();
            if (tid == 0) {
                long long cc = 0, ll = 0;
                for (int k = 0; k < NW; ++k) {
                    cc += h.red[0][k];
                    ll += h.red[1][k];
                }
                const unsigned long long o = atomicAdd(p.pool_cursor, (unsigned long long)cc);
                const bool fits = o + (unsigned long long)cc <= (unsigned long long)p.pool_cap;
                h.off = fits ? (long long)o : -1ll;
                if (fits) {
                    p.fill_count[i] = (int32_t)cc;
                    p.ucut[i] = (int32_t)ll;
                } else {
                    h.fail = 1;
                }
            }
            __syncthreads();
            if (!h.fail) {
                int32_t *dst = p.pool + h.off;
                long long run = 0;
                for (int w0 = 0; w0 < nw; w0 += NT) {
                    const int w = w0 + tid;
                    uint32_t x = w < nw ? bm[w] : 0u;
                    long long tot;
                    long long pos = run + scan_excl(__popc(x), h, &tot);
                    for (; x; x &= x - 1, ++pos) dst[pos] = (w << 5) + __ffs(x) - 1;
                    run += tot;
                }
                __threadfence();
                __syncthreads();
                if (tid == 0) st_release(p.row_off + i, h.off);
            }
        }
        if (h.fail && tid == 0) {
            p.fail_list[atomicAdd(p.fail_cnt, 1ull)] = i;
            st_release(p.row_off + i, -1);
        }
        // ---- fill(:) = 0 for the next row (L115)
        __syncthreads();
        for (int w = tid; w < nw; w += NT) bm[w] = 0;
        __syncthreads();
    }
    if (tid == 0 && p.stats) {
        atomicAdd(p.stats + 0, n_read);
        atomicAdd(p.stats + 1, n_rounds);
        atomicAdd(p.stats + 2, n_waits);
    }
}

// ascending bitonic sort of list[0..min(*cnt, max)) in shared memory (max <= kMergeSortMax)
__global__ void __launch_bounds__(1024) k_sort_list(int32_t *list, const unsigned long long *cnt,
                                                    int32_t max)
{
    __shared__ int32_t a[kMergeSortMax];
    const int m = (int)min(*cnt, (unsigned long long)max);
    if (m <= 1) return;
    int sz = 1;
    while (sz < m) sz <<= 1;
    for (int k = threadIdx.x; k < sz; k += blockDim.x) a[k] = k < m ? list[k] : INT_MAX;
    __syncthreads();
    for (int kk = 2; kk <= sz; kk <<= 1)
        for (int j = kk >> 1; j > 0; j >>= 1) {
            for (int x = threadIdx.x; x < sz; x += blockDim.x) {
                const int y = x ^ j;
                if (y > x) {
                    const bool up = (x & kk) == 0;
                    const int32_t u = a[x], v = a[y];
                    if ((u > v) == up) {
                        a[x] = v;
                        a[y] = u;
                    }
                }
            }
            __syncthreads();
        }
    for (int k = threadIdx.x; k < m; k += blockDim.x) list[k] = a[k];
}

}  // namespace

size_t merge_smem_bytes(int n, bool smem_bitmap, int q)
{
    size_t b = kHdrBytes + 2 * (size_t)NT * sizeof(long long) + 2 * (size_t)q * sizeof(int32_t);
    if (smem_bitmap) b += (size_t)((n + 31) / 32) * sizeof(uint32_t);
    return (b + 15) & ~(size_t)15;
}

cudaError_t merge_configure(size_t smem)
{
    cudaError_t e = cudaFuncSetAttribute(k_merge_rows<true>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return cudaFuncSetAttribute(k_merge_rows<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)smem);
}

cudaError_t merge_sort_list(int32_t *list, const unsigned long long *cnt, int32_t max,
                            cudaStream_t s)
{
    k_sort_list<<<1, 1024, 0, s>>>(list, cnt, max);
    return cudaGetLastError();
}

cudaError_t merge_launch(const MergeParams &p, bool smem_bitmap, int grid, size_t smem,
                         cudaStream_t s)
{
    static_assert(sizeof(MHdr) <= kHdrBytes, "merge header too large");
    if (smem_bitmap)
        k_merge_rows<true><<<grid, NT, smem, s>>>(p);
    else
        k_merge_rows<false><<<grid, NT, smem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace lusym
