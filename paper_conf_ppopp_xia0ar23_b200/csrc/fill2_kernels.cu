// fill2 traversal kernels (S3 count / S6 emit) for sm_100a.
//
// One CTA owns one source row at a time ("symbolic factorization from each
// source row is independent") and pulls rows from a device counter, heaviest (largest id)
// first (L272: per-row work grows with the row id).  Per row it runs Algorithm 1 (L110-161):
//
//   seed    : mark src and every v in A(src,:)                                  (L116-129)
//   loop    : thresholds in strictly increasing order (L130) — taken as a sorted WINDOW of the
//             marked-but-unprocessed vertices in (ptr, src) (reading R4), and
//             * "simple" thresholds (all below-neighbours already visited) are scanned in
//               parallel: their unvisited above-neighbours are pattern entries (reading R5b);
//             * the smallest non-simple threshold t0 runs a level-synchronous BFS over
//               unvisited vertices < t0 (L131-158); order inside a level is free (R5).
//   output  : L(src,:) = thresholds in the order the pointer passes them (already sorted),
//             U(src,:) = visited bits in (src, n) scanned upward (sorted), diagonal iff in A.
//
// Visited state: 1 bit per vertex, in shared memory when n/8 bytes fit next to the frontier
// queues (else in an HBM slot per CTA, reading R3/R25: zeroed per pass, cleared per row over
// the dirty word range only).  Frontier queues live in shared memory and spill to a per-CTA
// HBM region (capacity n).  Adjacency is read through an ELL-W copy of A without the diagonal
// (one 16/32-byte load per scanned vertex); vertices of larger degree are scanned by a whole
// warp from A's CSR.
#include "internal.h"

#include <climits>

namespace lusym {
namespace {

constexpr unsigned kFull = 0xffffffffu;

struct Hdr {
    int row, minseed, diag, tns, newmin, ucnt, lmin, lmax;
    int cnt[3];
    int pad;
    long long stage_off;
    int scan[40];
};
static_assert(sizeof(Hdr) <= kHdrBytes, "header too large");

template <int NT>
__device__ __forceinline__ int block_scan_excl(int x, int *s, int &total)
{
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(kFull, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) s[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        int v = lane < NW ? s[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(kFull, v, o);
            if (lane >= o) v += y;
        }
        if (lane < NW) s[lane] = v;
    }
    __syncthreads();
    total = s[NW - 1];
    const int r = (wid ? s[wid - 1] : 0) + inc - x;
    __syncthreads();
    return r;
}

template <bool GB>
__device__ __forceinline__ uint32_t bm_word(const uint32_t *bm, int w)
{
    if (GB) return __ldcg(bm + w);
    return bm[w];
}

template <bool GB>
__device__ __forceinline__ bool visited(const uint32_t *bm, int v)
{
    return (bm_word<GB>(bm, v >> 5) >> (v & 31)) & 1u;
}

// test-and-set (reading R26): true iff this call set the bit
__device__ __forceinline__ bool mark(uint32_t *bm, int v)
{
    const uint32_t b = 1u << (v & 31);
    return !(atomicOr(bm + (v >> 5), b) & b);
}

template <int W>
__device__ __forceinline__ void load_nb(const int32_t *ell, int f, int (&nb)[W])
{
    const int4 *p = reinterpret_cast<const int4 *>(ell + (size_t)f * W);
    const int4 a = __ldg(p);
    nb[0] = a.x; nb[1] = a.y; nb[2] = a.z; nb[3] = a.w;
    if constexpr (W == 8) {
        const int4 b = __ldg(p + 1);
        nb[4] = b.x; nb[5] = b.y; nb[6] = b.z; nb[7] = b.w;
    }
}

__device__ __forceinline__ int64_t heavy_off(int lo, int hi)
{
    return (int64_t)(uint32_t)lo | ((int64_t)hi << 32);
}

// warp-aggregated append to the next frontier (smem, spilling to HBM past q entries)
__device__ __forceinline__ void push(bool pred, int w, int *cnt, int32_t *NF, int32_t *gNF, int q,
                                     unsigned long long &spills)
{
    const unsigned b = __ballot_sync(kFull, pred);
    if (b == 0) return;
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(cnt, __popc(b));
    base = __shfl_sync(kFull, base, leader);
    if (pred) {
        const int pos = base + __popc(b & ((1u << lane) - 1u));
        if (pos < q) {
            NF[pos] = w;
        } else {
            gNF[pos] = w;
            ++spills;
        }
    }
}

// Sorted list of the set bits in [lo, hi), at most cap of them, into out[]. Block-uniform.
template <int NT, bool GB>
__device__ int collect(const uint32_t *bm, int lo, int hi, int32_t *out, int cap, int *sscan)
{
    if (lo >= hi) return 0;
    const int wlo = lo >> 5, whi = (hi - 1) >> 5;
    int count = 0;
    for (int wb = wlo; wb <= whi; wb += NT) {
        const int w = wb + (int)threadIdx.x;
        uint32_t word = 0;
        if (w <= whi) {
            word = bm_word<GB>(bm, w);
            if (w == wlo) word &= kFull << (lo & 31);
            if (w == whi) {
                const int hb = (hi - 1) & 31;
                word &= (hb == 31) ? kFull : ((2u << hb) - 1u);
            }
        }
        int total;
        int pos = count + block_scan_excl<NT>(__popc(word), sscan, total);
        while (word != 0 && pos < cap) {
            out[pos++] = (w << 5) + (__ffs(word) - 1);
            word &= word - 1;
        }
        count += total;
        if (count >= cap) {
            count = cap;
            break;
        }
    }
    __syncthreads();
    return count;
}

// Write the set bits in [lo, hi) in increasing order to dst[0..) (global).  Block-uniform.
template <int NT, bool GB>
__device__ void emit_bits(const uint32_t *bm, int lo, int hi, int32_t *dst, int *sscan)
{
    if (lo >= hi) return;
    const int wlo = lo >> 5, whi = (hi - 1) >> 5;
    int count = 0;
    for (int wb = wlo; wb <= whi; wb += NT) {
        const int w = wb + (int)threadIdx.x;
        uint32_t word = 0;
        if (w <= whi) {
            word = bm_word<GB>(bm, w);
            if (w == wlo) word &= kFull << (lo & 31);
            if (w == whi) {
                const int hb = (hi - 1) & 31;
                word &= (hb == 31) ? kFull : ((2u << hb) - 1u);
            }
        }
        int total;
        int pos = count + block_scan_excl<NT>(__popc(word), sscan, total);
        while (word != 0) {
            dst[pos++] = (w << 5) + (__ffs(word) - 1);
            word &= word - 1;
        }
        count += total;
    }
}

struct RowAcc {
    int ucnt, lmin, lmax;
    unsigned long long te, sv, spills;
};

// Level-synchronous BFS from threshold t0 over unvisited vertices < t0 (Alg. 1).
template <int NT, int W, bool GB>
__device__ void bfs(const Fill2Params &p, Hdr &h, uint32_t *bm, int32_t *qA, int32_t *qB,
                    int32_t *gA, int32_t *gB, const int i, const int t0, RowAcc &a)
{
    const int tid = threadIdx.x, lane = tid & 31;
    int32_t *F = qA, *NF = qB, *gF = gA, *gNF = gB;
    if (tid == 0) {
        F[0] = t0;
        h.cnt[0] = 1;
        h.cnt[1] = 0;
        h.cnt[2] = 0;
    }
    __syncthreads();
    int fsize = 1;
    for (int lev = 0;; ++lev) {
        int *nsz = &h.cnt[(lev + 1) % 3];
        if (tid == 0) h.cnt[(lev + 2) % 3] = 0;
        for (int base = 0; base < fsize; base += NT) {
            const int k = base + tid;
            const bool valid = k < fsize;
            int nb[W];
#pragma unroll
            for (int s = 0; s < W; ++s) nb[s] = -1;
            bool heavy = false;
            if (valid) {
                const int f = k < p.q ? F[k] : __ldcg(gF + k);
                load_nb<W>(p.ell, f, nb);
                heavy = nb[0] == kHeavy;
            }
            // light vertex: test-and-set its <= W neighbours, remember the new frontier ones
            uint32_t frm = 0;
            if (valid && !heavy) {
                ++a.sv;
#pragma unroll
                for (int s = 0; s < W; ++s) {
                    const int w = nb[s];
                    if (w >= 0 && !visited<GB>(bm, w) && mark(bm, w)) {
                        if (w < t0) {
                            frm |= 1u << s;
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
            }
            // one warp-aggregated append for all new frontier vertices of the warp
            {
                const int c = __popc(frm);
                int inc = c;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int y = __shfl_up_sync(kFull, inc, o);
                    if (lane >= o) inc += y;
                }
                const int total = __shfl_sync(kFull, inc, 31);
                if (total) {
                    int wbase = 0;
                    if (lane == 31) wbase = atomicAdd(nsz, total);
                    wbase = __shfl_sync(kFull, wbase, 31);
                    int pos = wbase + inc - c;
#pragma unroll
                    for (int s = 0; s < W; ++s) {
                        if (frm & (1u << s)) {
                            const int w = nb[s];
                            a.lmin = min(a.lmin, w);
                            if (pos < p.q) {
                                NF[pos] = w;
                            } else {
                                gNF[pos] = w;
                                ++a.spills;
                            }
                            ++pos;
                        }
                    }
                }
            }
            unsigned hm = __ballot_sync(kFull, valid && heavy);
            while (hm) {
                const int src = __ffs(hm) - 1;
                hm &= hm - 1;
                const int len = __shfl_sync(kFull, nb[1], src);
                const int64_t off =
                    heavy_off(__shfl_sync(kFull, nb[2], src), __shfl_sync(kFull, nb[3], src));
                if (lane == 0) {
                    a.te += len;
                    ++a.sv;
                }
                for (int eb = 0; eb < len; eb += 32) {
                    const int e = eb + lane;
                    bool fr = false;
                    int w = -1;
                    if (e < len) {
                        w = __ldg(p.ci + off + e);
                        if (!visited<GB>(bm, w) && mark(bm, w)) {
                            if (w < t0) {
                                fr = true;
                                a.lmin = min(a.lmin, w);
                            } else if (w > i) {
                                ++a.ucnt;
                                a.lmax = max(a.lmax, w);
                            }
                        }
                    }
                    push(fr, w, nsz, NF, gNF, p.q, a.spills);
                }
            }
        }
        __syncthreads();
        fsize = *nsz;
        if (fsize == 0) break;
        int32_t *t = F; F = NF; NF = t;
        t = gF; gF = gNF; gNF = t;
    }
}

// MODE: kCount (symbolic_1, counts only), kStage (counts + rows staged into the HBM pool, so
// symbolic_2 becomes a placement copy), kEmit (symbolic_2 by traversal, into the final CSR).
template <int NT, int W, int MODE, bool GB>
__global__ void __launch_bounds__(NT) fill2_kernel(const Fill2Params p)
{
    extern __shared__ __align__(16) unsigned char smem[];
    Hdr &h = *reinterpret_cast<Hdr *>(smem);
    int32_t *qA = reinterpret_cast<int32_t *>(smem + kHdrBytes);
    int32_t *qB = qA + p.q;
    uint32_t *bm;
    if constexpr (GB)
        bm = p.gbitmap + (size_t)blockIdx.x * p.gbitmap_stride;
    else
        bm = reinterpret_cast<uint32_t *>(qB + p.q);
    int32_t *gA = p.gspill + (size_t)blockIdx.x * 2 * p.spill_cap;
    int32_t *gB = gA + p.spill_cap;
    const int tid = threadIdx.x, lane = tid & 31;
    if constexpr (!GB)
        for (int w = tid; w < p.nw; w += NT) bm[w] = 0;

    RowAcc a;
    a.te = a.sv = a.spills = 0;
    const int nrows = p.row_end - p.row_begin;
    for (;;) {
        if (tid == 0) {
            const unsigned long long c = atomicAdd(p.row_counter, 1ull);
            int r = -1;
            if (p.row_list) {
                if (c < (unsigned long long)p.list_len) r = p.row_list[c];
            } else if (c < (unsigned long long)nrows) {
                r = p.descending ? p.row_end - 1 - (int)c : p.row_begin + (int)c;
            }
            h.row = r;
            h.minseed = r;
            h.diag = 0;
            h.ucnt = 0;
            h.lmin = r;
            h.lmax = r;
        }
        __syncthreads();
        const int i = h.row;
        if (i < 0) break;
        a.ucnt = 0;
        a.lmin = i;
        a.lmax = i;

        // ---- seed: fill(src) = src; for v in A(src,:) fill(v) = src  (L116-129)
        const int64_t rb = p.rp[i], re = p.rp[i + 1];
        for (int64_t k = rb + tid; k < re; k += NT) {
            const int v = __ldg(p.ci + k);
            ++a.te;
            atomicOr(bm + (v >> 5), 1u << (v & 31));
            if (v < i) {
                atomicMin(&h.minseed, v);
                a.lmin = min(a.lmin, v);
            } else if (v > i) {
                ++a.ucnt;
                a.lmax = max(a.lmax, v);
            } else {
                h.diag = 1;
            }
        }
        if (tid == 0) atomicOr(bm + (i >> 5), 1u << (i & 31));
        __syncthreads();

        int ptr = h.minseed - 1;  // every unprocessed threshold is > ptr
        int Lcnt = 0;
        // destination of the L entries (written in threshold order, i.e. sorted)
        int32_t *ldst = nullptr;
        int64_t lcap = 0;
        if constexpr (MODE == kEmit) {
            const int64_t obase = p.rp_lu[i];
            ldst = p.ci_lu + obase;
            lcap = p.rp_lu[i + 1] - obase;
        } else if constexpr (MODE == kStage) {
            ldst = p.stg + (size_t)blockIdx.x * p.spill_cap;
            lcap = p.n;
        }
        // ---- thresholds in increasing order (L130)
        for (;;) {
            const int wc = collect<NT, GB>(bm, ptr + 1, i, qA, p.wcap, h.scan);
            if (wc == 0) break;
            if (tid == 0) {
                h.tns = INT_MAX;
                h.newmin = INT_MAX;
            }
            __syncthreads();
            int nm = INT_MAX;
            for (int base = 0; base < wc; base += NT) {
                const int k = base + tid;
                const bool valid = k < wc;
                const int t = valid ? qA[k] : 0;
                int nb[W];
#pragma unroll
                for (int s = 0; s < W; ++s) nb[s] = -1;
                bool heavy = false;
                if (valid) {
                    load_nb<W>(p.ell, t, nb);
                    heavy = nb[0] == kHeavy;
                }
                if (valid && !heavy) {
                    ++a.sv;
                    bool simple = true;
#pragma unroll
                    for (int s = 0; s < W; ++s) {
                        const int w = nb[s];
                        if (w >= 0 && w < t && !visited<GB>(bm, w)) simple = false;
                    }
                    if (!simple) {
                        atomicMin(&h.tns, t);
                    } else {
#pragma unroll
                        for (int s = 0; s < W; ++s) {
                            const int w = nb[s];
                            if (w > t && !visited<GB>(bm, w) && mark(bm, w)) {
                                if (w < i) {
                                    nm = min(nm, w);
                                } else {
                                    ++a.ucnt;
                                    a.lmax = max(a.lmax, w);
                                }
                            }
                        }
                    }
                }
                unsigned hm = __ballot_sync(kFull, valid && heavy);
                while (hm) {
                    const int src = __ffs(hm) - 1;
                    hm &= hm - 1;
                    const int tt = __shfl_sync(kFull, t, src);
                    const int len = __shfl_sync(kFull, nb[1], src);
                    const int64_t off = heavy_off(__shfl_sync(kFull, nb[2], src),
                                                  __shfl_sync(kFull, nb[3], src));
                    bool ok = true;
                    for (int e = lane; e < len; e += 32) {
                        const int w = __ldg(p.ci + off + e);
                        if (w < tt && !visited<GB>(bm, w)) ok = false;
                    }
                    ok = __all_sync(kFull, ok);
                    if (lane == 0) {
                        a.te += len;
                        ++a.sv;
                    }
                    if (!ok) {
                        if (lane == 0) atomicMin(&h.tns, tt);
                    } else {
                        for (int e = lane; e < len; e += 32) {
                            const int w = __ldg(p.ci + off + e);
                            if (w > tt && !visited<GB>(bm, w) && mark(bm, w)) {
                                if (w < i) {
                                    nm = min(nm, w);
                                } else {
                                    ++a.ucnt;
                                    a.lmax = max(a.lmax, w);
                                }
                            }
                        }
                    }
                }
            }
            if (nm != INT_MAX) atomicMin(&h.newmin, nm);
            __syncthreads();
            const int tns = h.tns;
            const int m = min(tns, h.newmin);
            const int last = qA[wc - 1];
            if (m > last) {  // the whole window is processed
                if constexpr (MODE != kCount)
                    for (int k = tid; k < wc; k += NT)
                        if (Lcnt + k < lcap) ldst[Lcnt + k] = qA[k];
                Lcnt += wc;
                ptr = last;
                __syncthreads();
                continue;
            }
            // window elements below m are processed; m is the smallest pending threshold
            int lo = 0, hi = wc;
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (qA[mid] < m) lo = mid + 1; else hi = mid;
            }
            const int e = lo;
            if constexpr (MODE != kCount)
                for (int k = tid; k < e; k += NT)
                    if (Lcnt + k < lcap) ldst[Lcnt + k] = qA[k];
            Lcnt += e;
            if (m == tns) {  // smallest pending threshold needs a below-exploration
                if constexpr (MODE != kCount)
                    if (tid == 0 && Lcnt < lcap) ldst[Lcnt] = m;
                Lcnt += 1;
                __syncthreads();
                bfs<NT, W, GB>(p, h, bm, qA, qB, gA, gB, i, m, a);
                ptr = m;
            } else {  // a simple threshold marked a new pending one below the window's rest
                ptr = m - 1;
                __syncthreads();
            }
        }

        // ---- U part, diagonal, count / emission
        if (a.ucnt) atomicAdd(&h.ucnt, a.ucnt);
        if (a.lmin < i) atomicMin(&h.lmin, a.lmin);
        if (a.lmax > i) atomicMax(&h.lmax, a.lmax);
        __syncthreads();
        const int ucnt = h.ucnt, diag = h.diag, gmin = h.lmin, gmax = h.lmax;
        const int len = Lcnt + diag + ucnt;
        if constexpr (MODE == kCount) {
            if (tid == 0) p.fill_count[i] = len;
        } else if constexpr (MODE == kStage) {
            // reserve len entries of the pool; rows that do not fit are re-traversed by emit
            if (tid == 0) {
                p.fill_count[i] = len;
                const unsigned long long off = atomicAdd(p.pool_cursor, (unsigned long long)len);
                const bool fits = off + (unsigned long long)len <= (unsigned long long)p.pool_cap;
                h.stage_off = fits ? (long long)off : -1ll;
                p.row_off[i] = fits ? (int64_t)off : -1;
                if (!fits) p.unstaged[atomicAdd(p.unstaged_cnt, 1ull)] = i;
            }
            __syncthreads();
            const long long off = h.stage_off;
            if (off >= 0) {
                int32_t *dst = p.pool + off;
                for (int k = tid; k < Lcnt; k += NT) dst[k] = ldst[k];
                if (diag && tid == 0) dst[Lcnt] = i;
                emit_bits<NT, GB>(bm, i + 1, gmax + 1, dst + Lcnt + diag, h.scan);
            }
        } else {
            if (lcap != (int64_t)len) {
                if (tid == 0) atomicAdd(p.stats + kStatErr, 1ull);
            } else {
                if (diag && tid == 0) ldst[Lcnt] = i;
                emit_bits<NT, GB>(bm, i + 1, gmax + 1, ldst + Lcnt + diag, h.scan);
            }
        }
        // ---- clear the dirty word range (fill(:) = 0 for the next row, L115)
        for (int w = (gmin >> 5) + tid; w <= (gmax >> 5); w += NT) bm[w] = 0;
        __syncthreads();
    }

    // flush statistics
    unsigned long long te = a.te, sv = a.sv, sp = a.spills;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        te += __shfl_xor_sync(kFull, te, o);
        sv += __shfl_xor_sync(kFull, sv, o);
        sp += __shfl_xor_sync(kFull, sp, o);
    }
    if (lane == 0) {
        atomicAdd(p.stats + kStatEdges, te);
        atomicAdd(p.stats + kStatVerts, sv);
        if (sp) atomicAdd(p.stats + kStatSpills, sp);
    }
}

template <int NT, int W, bool GB>
cudaError_t launch_one(const Fill2Params &p, int mode, int grid, size_t smem, cudaStream_t s)
{
    if (mode == kCount)
        fill2_kernel<NT, W, kCount, GB><<<grid, NT, smem, s>>>(p);
    else if (mode == kStage)
        fill2_kernel<NT, W, kStage, GB><<<grid, NT, smem, s>>>(p);
    else
        fill2_kernel<NT, W, kEmit, GB><<<grid, NT, smem, s>>>(p);
    return cudaGetLastError();
}

template <int NT, int W, int MODE, bool GB>
cudaError_t configure_mode(size_t smem)
{
    cudaError_t e = cudaFuncSetAttribute(fill2_kernel<NT, W, MODE, GB>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    cudaFuncSetAttribute(fill2_kernel<NT, W, MODE, GB>,
                         cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    return cudaSuccess;
}

template <int NT, int W, bool GB>
cudaError_t configure_one(size_t smem)
{
    cudaError_t e = configure_mode<NT, W, kCount, GB>(smem);
    if (e == cudaSuccess) e = configure_mode<NT, W, kStage, GB>(smem);
    if (e == cudaSuccess) e = configure_mode<NT, W, kEmit, GB>(smem);
    return e;
}

template <int NT, int W, bool GB>
cudaError_t occupancy_one(size_t smem, int *occ)
{
    int a = 0, b = 0, c = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(
        &a, fill2_kernel<NT, W, kCount, GB>, NT, smem);
    if (e == cudaSuccess)
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, fill2_kernel<NT, W, kStage, GB>, NT,
                                                          smem);
    if (e == cudaSuccess)
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&c, fill2_kernel<NT, W, kEmit, GB>, NT,
                                                          smem);
    *occ = a < b ? a : b;
    *occ = *occ < c ? *occ : c;
    return e;
}

}  // namespace

size_t fill2_smem_bytes(int n, int q, bool global_bitmap)
{
    size_t b = kHdrBytes + 2 * (size_t)q * sizeof(int32_t);
    if (!global_bitmap) b += (size_t)((n + 31) / 32) * sizeof(uint32_t);
    return (b + 15) & ~(size_t)15;
}

#define LUSYM_DISPATCH(NTV, WV, GBV, CALL)                                                   \
    if (nt == NTV && w == WV && gb == GBV) return CALL;

cudaError_t fill2_configure(int nt, int w, bool gb, size_t smem)
{
#define CFG(NTV, WV, GBV) LUSYM_DISPATCH(NTV, WV, GBV, (configure_one<NTV, WV, GBV>(smem)))
    CFG(128, 4, false) CFG(128, 4, true) CFG(128, 8, false) CFG(128, 8, true)
    CFG(256, 4, false) CFG(256, 4, true) CFG(256, 8, false) CFG(256, 8, true)
    CFG(512, 4, false) CFG(512, 4, true) CFG(512, 8, false) CFG(512, 8, true)
    CFG(1024, 4, false) CFG(1024, 4, true) CFG(1024, 8, false) CFG(1024, 8, true)
#undef CFG
    return cudaErrorInvalidValue;
}

cudaError_t fill2_occupancy(int nt, int w, bool gb, size_t smem, int *occ)
{
#define OCC(NTV, WV, GBV) LUSYM_DISPATCH(NTV, WV, GBV, (occupancy_one<NTV, WV, GBV>(smem, occ)))
    OCC(128, 4, false) OCC(128, 4, true) OCC(128, 8, false) OCC(128, 8, true)
    OCC(256, 4, false) OCC(256, 4, true) OCC(256, 8, false) OCC(256, 8, true)
    OCC(512, 4, false) OCC(512, 4, true) OCC(512, 8, false) OCC(512, 8, true)
    OCC(1024, 4, false) OCC(1024, 4, true) OCC(1024, 8, false) OCC(1024, 8, true)
#undef OCC
    return cudaErrorInvalidValue;
}

cudaError_t fill2_launch(const Fill2Params &p, int nt, int w, int mode, bool gb, int grid,
                         size_t smem, cudaStream_t s)
{
#define LCH(NTV, WV, GBV)                                                                    \
    LUSYM_DISPATCH(NTV, WV, GBV, (launch_one<NTV, WV, GBV>(p, mode, grid, smem, s)))
    LCH(128, 4, false) LCH(128, 4, true) LCH(128, 8, false) LCH(128, 8, true)
    LCH(256, 4, false) LCH(256, 4, true) LCH(256, 8, false) LCH(256, 8, true)
    LCH(512, 4, false) LCH(512, 4, true) LCH(512, 8, false) LCH(512, 8, true)
    LCH(1024, 4, false) LCH(1024, 4, true) LCH(1024, 8, false) LCH(1024, 8, true)
#undef LCH
    return cudaErrorInvalidValue;
}

}  // namespace lusym
