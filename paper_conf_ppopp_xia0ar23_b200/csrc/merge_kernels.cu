// Deferred rows of the count pass, finished by row-merge closure over staged rows (reading G8,
// DESIGN.md §2).
//
// Theorem 1 split at the largest intermediate vertex t of a path i -> j: the
// part i -> t has intermediates < t, the part t -> j too, so for j != i
//     (i,j) in P  iff  A(i,j) != 0  or  (i,t) in P and (t,j) in P for some t < min(i,j).
// Row i of L+U is therefore the least set S with S ⊇ A(i,:) and S ⊇ U_t = {j > t : (t,j) in P}
// for every t in S with t < i (the diagonal comes from A only, reading R7).  A least fixed
// point does not depend on the order its members are expanded in, so a whole frontier of new
// members t < i is expanded at once: there is no serial chain of increasing thresholds
// (Alg. 1), which on circuit matrices with hubs ordered last makes a single row cost
// 10^5 dependent threshold windows.  Rows t are read from the staging pool the count pass
// filled (their strict-U part starts ucut[t] entries into the row).
//
// One row is processed by a cluster of G CTAs (kMergeCluster) whose shared memories hold the
// row's visited bitmap in G slices (distributed shared memory, test-and-set by DSMEM atomics),
// or by one CTA with the whole bitmap in shared memory or in an HBM slot.  Each CTA expands
// the members it discovered itself; cluster barriers end a round.
//
// Rows are claimed in increasing order.  A member t that is itself a deferred row still in
// progress is set aside until its cluster publishes it (row_off[t] >= 0, release/acquire); the
// smallest unfinished claimed row never waits, so the resident grid always progresses.  A row
// that cannot be finished (a row it needs is unstaged, or the pool is full) is listed for the
// fill2 fallback launch that follows.
#include "internal.h"

#include <climits>
#include <cstdio>
#include <cooperative_groups.h>
#include <map>
#include <mutex>
#include <tuple>

namespace cg = cooperative_groups;

namespace lusym {
namespace {

constexpr int NT = kMergeNT;
constexpr int NW = NT / 32;
#ifndef LUSYM_MERGE_KU
#define LUSYM_MERGE_KU 1  // windows in flight per warp (A/B on cfg3: 1 = 14.8 ms tail, 2 = 15.2, 4 = 15.2, 8 = 15.4)
#endif
#ifndef LUSYM_MERGE_PROF
#define LUSYM_MERGE_PROF 0
#endif
#ifndef LUSYM_MERGE_HASH  // cluster mode: new members spread over the ranks by a hash of their id
#define LUSYM_MERGE_HASH 1
#endif
#ifndef LUSYM_MERGE_LDCG  // expansion: pool entries read through L2 only (ld.global.cg)
#define LUSYM_MERGE_LDCG 0
#endif
#ifndef LUSYM_MERGE_BATCH  // expansion: the kU windows' visited words loaded before any atomic
#define LUSYM_MERGE_BATCH 0
#endif
constexpr int kU = LUSYM_MERGE_KU;  // pool loads in flight per thread
constexpr int kSent = 64;  // sentinel starts past the last segment

struct MHdr {
    int row, diag, fail, nwait;
    int cnt[2];
    int tn, tw, tf, tdiag;  // cluster totals of the round (thread 0 -> block)
    long long off;
    long long part_c, part_lo;
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

// block sums of two 64-bit values (valid in every thread)
__device__ __forceinline__ void block_sum2(long long &a, long long &b, MHdr &h)
{
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        a += __shfl_xor_sync(0xffffffffu, a, o);
        b += __shfl_xor_sync(0xffffffffu, b, o);
    }
    if ((threadIdx.x & 31) == 0) {
        h.red[0][threadIdx.x >> 5] = a;
        h.red[1][threadIdx.x >> 5] = b;
    }
    __syncthreads();
    a = b = 0;
#pragma unroll
    for (int k = 0; k < NW; ++k) {
        a += h.red[0][k];
        b += h.red[1][k];
    }
    __syncthreads();
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

// Cluster mode: a new member goes to the frontier of the rank a hash of its id picks (DSMEM
// atomics on that rank's counter, stores into its queue), not to the discovering rank's: the
// ranks then expand equal shares of the next round instead of waiting at the cluster barrier
// for the rank that happened to discover the most (cfg3's largest hub: 54% of the tail's stall
// samples were cluster barrier waits).
template <int MODE>
__device__ __forceinline__ void q_push_hashed(bool pred, int32_t w, int *cnt_local,
                                              int32_t *sq_local, int32_t *gq_rank0, int64_t gstride,
                                              int rank, int g, int q)
{
    const unsigned any = __ballot_sync(0xffffffffu, pred);
    if (!any) return;
    const int lane = threadIdx.x & 31;
    const int dst = pred ? (int)((((uint32_t)w * 2654435761u) >> 16) % (uint32_t)g) : -1;
    auto cl = cg::this_cluster();
    for (int r = 0; r < g; ++r) {
        const unsigned b = __ballot_sync(0xffffffffu, dst == r);
        if (!b) continue;
        const int leader = __ffs(b) - 1;
        int base = 0;
        if (lane == leader) {
            int *c = r == rank ? cnt_local : cl.map_shared_rank(cnt_local, r);
            base = atomicAdd(c, __popc(b));
        }
        base = __shfl_sync(0xffffffffu, base, leader);
        if (dst == r) {
            const int pos = base + __popc(b & ((1u << lane) - 1u));
            if (pos < q) {
                int32_t *d = r == rank ? sq_local : cl.map_shared_rank(sq_local, r);
                d[pos] = w;
            } else {
                gq_rank0[(int64_t)r * gstride + pos] = w;
            }
        }
    }
}

// The row's visited bitmap: whole in this CTA (shared memory or HBM slot), or sliced over the
// cluster, word w in rank w >> sh at local index w & (wpc - 1).
template <bool CL>
struct Bits {
    uint32_t *w;  // local words
    int sh;       // log2(words per CTA) (cluster)
    int rank, g;  // cluster rank and size (1 / 0 without a cluster)
    int lo, hi;   // local word range [lo, hi) in global word numbering

    __device__ __forceinline__ uint32_t *word(int gw) const
    {
        if constexpr (!CL) return w + gw;
        const int r = gw >> sh;
        uint32_t *base = w + (gw & ((1 << sh) - 1));
        return r == rank ? base : cg::this_cluster().map_shared_rank(base, r);
    }
    uint32_t *filt = nullptr;  // cluster mode: bits this CTA has seen set in other ranks' words

    // test-and-set of bit v; true iff this call set it.  A remote word's test first looks at
    // the CTA's filter: bits are only ever set during a row, so a bit seen set (in a word this
    // CTA read or set earlier) is set, and the DSMEM round trip is skipped; every remote word
    // read or atomically modified is OR-ed into the filter.
    __device__ __forceinline__ bool tas(int v) const
    {
        const uint32_t b = 1u << (v & 31);
        const int gw = v >> 5;
        if constexpr (CL) {
            const int r = gw >> sh;
            if (r != rank && filt) {
                if (filt[gw] & b) return false;
                uint32_t *p = cg::this_cluster().map_shared_rank(w + (gw & ((1 << sh) - 1)), r);
                const uint32_t cur = *p;
                if (cur & b) {
                    atomicOr(filt + gw, cur);
                    return false;
                }
                const uint32_t old = atomicOr(p, b);
                atomicOr(filt + gw, old | b);
                return !(old & b);
            }
        }
        uint32_t *p = word(gw);
        if (*p & b) return false;
        return !(atomicOr(p, b) & b);
    }
};

__device__ __forceinline__ void csync_impl(bool cl)
{
    if (cl) cg::this_cluster().sync(); else __syncthreads();
}

// MODE: 0 = one CTA, bitmap in shared memory; 1 = one CTA, bitmap in an HBM slot;
//       2 = a cluster of G CTAs, bitmap sliced over their shared memories
template <int MODE>
__global__ void __launch_bounds__(NT, 1) k_merge_rows(const MergeParams p, int sh)
{
    constexpr bool CL = MODE == 2;
    extern __shared__ __align__(16) unsigned char smem[];
    MHdr &h = *reinterpret_cast<MHdr *>(smem);
    // compacted frontier segments of one block of members: pool offset and flat start
    long long *c_off = reinterpret_cast<long long *>(smem + kHdrBytes);    // [NT]
    long long *c_start = c_off + NT;                                        // [NT + kSent]
    int32_t *sq = reinterpret_cast<int32_t *>(c_start + NT + kSent);       // 2 x q
    const int nw = (p.n + 31) >> 5;
    Bits<CL> bm;
    bm.sh = sh;
    if constexpr (CL) {
        bm.rank = (int)cg::this_cluster().block_rank();
        bm.g = (int)cg::this_cluster().num_blocks();
        bm.w = reinterpret_cast<uint32_t *>(sq + 2 * p.q);
        bm.lo = min(nw, bm.rank << sh);
        bm.hi = min(nw, (bm.rank + 1) << sh);
    } else {
        bm.rank = 0;
        bm.g = 1;
        bm.w = MODE == 0 ? reinterpret_cast<uint32_t *>(sq + 2 * p.q)
                         : p.gbitmap + (size_t)blockIdx.x * p.gb_stride;
        bm.lo = 0;
        bm.hi = nw;
    }
    uint32_t *lw = CL ? bm.w - bm.lo : bm.w;  // local words by global word index
    int32_t *gq0 = p.spill + (size_t)blockIdx.x * 2 * p.spill_cap;
    int32_t *wait = p.wait + (size_t)blockIdx.x * p.list_max;
    const int tid = threadIdx.x;
    if constexpr (CL) {
        bm.filt = p.cl_filter ? bm.w + (1 << sh) : nullptr;
        for (int w = tid; w < p.cl_filter; w += NT) bm.filt[w] = 0;
    }
    const int nlist = (int)min(*p.list_cnt, (unsigned long long)p.list_max);
    if (MODE != 1)
        for (int w = bm.lo + tid; w < bm.hi; w += NT) lw[w] = 0;
    unsigned long long n_read = 0, n_rounds = 0, n_waits = 0;  // thread 0 of rank 0
    for (;;) {
        if (tid == 0) {
            h.diag = 0;
            h.fail = 0;
            h.nwait = 0;
            h.cnt[0] = h.cnt[1] = 0;
            if (bm.rank == 0) {
                const unsigned long long c = atomicAdd(p.counter, 1ull);
                h.row = c < (unsigned long long)nlist ? p.list[c] : -1;
            }
        }
        csync_impl(CL);
        if constexpr (CL) {
            if (tid == 0 && bm.rank != 0) h.row = cg::this_cluster().map_shared_rank(&h, 0)->row;
            // no CTA may exit (on the final claim, -1) while another still reads its shared
            // memory: a second barrier after the read of rank 0's claim
            cg::this_cluster().sync();
        }
        const int i = h.row;
        if (i < 0) break;
#if LUSYM_MERGE_PROF
        long long prof_setup = 0, prof_expand = 0, prof_tiles = 0, prof_entries = 0;
        unsigned long long t_claim = 0, t_firstwait = 0, t_lastwait = 0, rows_r = 0, nwaits_r = 0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_claim));
#endif
        // ---- seed: S = A(i,:); members t < i form the first frontier (entries split by rank)
        if (tid == 0 && bm.rank == 0) atomicOr(bm.word(i >> 5), 1u << (i & 31));
        csync_impl(CL);
        {
            const int64_t rb = p.rp[i], re = p.rp[i + 1];
            for (int64_t b0 = rb + (int64_t)bm.rank * NT; b0 < re; b0 += (int64_t)bm.g * NT) {
                const int64_t e = b0 + tid;
                int v = -1;
                bool fr = false;
                if (e < re) {
                    v = __ldg(p.ci + e);
                    if (v == i) h.diag = 1;
                    else if (bm.tas(v)) fr = v < i;
                }
                q_push(fr, v, &h.cnt[0], sq, gq0, p.q);
            }
        }
        __syncthreads();
        int cur = 0;
        int diag = 0, fail = 0;
        for (;;) {
            // cluster totals of the frontier in buffer cur, the wait lists and failures
            csync_impl(CL);
            if (tid == 0) {
                int tn = h.cnt[cur], tw = h.nwait, tf = h.fail, td = h.diag;
                if constexpr (CL)
                    for (int r = 0; r < bm.g; ++r)
                        if (r != bm.rank) {
                            const MHdr *o = cg::this_cluster().map_shared_rank(&h, r);
                            tn += o->cnt[cur];
                            tw += o->nwait;
                            tf |= o->fail;
                            td |= o->diag;
                        }
                h.tn = tn;
                h.tw = tw;
                h.tf = tf;
                h.tdiag = td;
            }
            __syncthreads();
            const int tn = h.tn, tw = h.tw;
            fail = h.tf;
            diag = h.tdiag;
            if constexpr (CL) cg::this_cluster().sync();  // everyone has read the counters
            if (fail) break;
            if (tn == 0) {
                if (tw == 0) break;
                // every member left is a deferred row still in progress: wait for them (each
                // was claimed before row i by a running cluster), then expand them
                const int nwt = h.nwait;
#if LUSYM_MERGE_PROF
                if (!t_firstwait) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_firstwait));
                nwaits_r += nwt;
#endif
                for (int k = tid; k < nwt; k += NT) {
                    const int t = wait[k];
                    while (ld_acquire(p.row_off + t) == kRowDeferred) __nanosleep(200);
                }
#if LUSYM_MERGE_PROF
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_lastwait));
#endif
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
                continue;
            }
            const int nxt = cur ^ 1;
            const int fsize = h.cnt[cur];
            const int32_t *fq = sq + cur * p.q, *gfq = gq0 + (size_t)cur * p.spill_cap;
            int32_t *nq = sq + nxt * p.q, *gnq = gq0 + (size_t)nxt * p.spill_cap;
            for (int base = 0; base < fsize; base += NT) {
#if LUSYM_MERGE_PROF
                long long c_t0 = clock64();
#endif
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
                // compact the non-empty segments (strictly increasing starts): one scan of
                // (len << 11 | nonempty)
                long long total;
                const long long st = scan_excl((len << 11) | (len > 0 ? 1 : 0), h, &total);
                const int nsrc = (int)(total & 2047);
                const long long E = total >> 11;
                if (len > 0) {
                    c_start[st & 2047] = st >> 11;
                    c_off[st & 2047] = off;
                }
                if (tid < kSent) c_start[nsrc + tid] = LLONG_MAX;
                __syncthreads();
                if (tid == 0) n_read += (unsigned long long)E;
#if LUSYM_MERGE_PROF
                long long c_t1 = clock64();
                if (tid == 0) prof_setup += c_t1 - c_t0;
#endif
                // each warp expands a contiguous chunk of the E flat positions, 32 at a time: one
                // binary search for the chunk's first owner, then the owner of lane l of a window
                // [p, p+32) is that window's owner plus the segments starting in (p, p+l]
                // (one OR-reduction of 32 start bits, no per-entry search)
                const int wid = tid >> 5, lane = tid & 31;
                const long long C = ((E + NW - 1) / NW + 31) & ~31ll;
                long long pw = (long long)wid * C;
                const long long pend = min(E, pw + C);
                if (pw < pend) {
                    int src = 0;
#pragma unroll
                    for (int step = NT / 2; step >= 1; step >>= 1)
                        if (src + step < nsrc && c_start[src + step] <= pw) src += step;
                    while (pw < pend) {
                        int jv[kU];
#pragma unroll
                        for (int u = 0; u < kU; ++u) {
                            jv[u] = -1;
                            if (pw < pend) {
                                const long long sn = c_start[src + 1 + lane];
                                const unsigned bit = sn < pw + 32 ? 1u << (int)(sn - pw) : 0u;
                                const unsigned mask = __reduce_or_sync(0xffffffffu, bit);
                                const int my = src + __popc(mask & ((2u << lane) - 1u));
                                if (pw + lane < pend)
                                    jv[u] = LUSYM_MERGE_LDCG
                                                ? __ldcg(p.pool + c_off[my] + (pw + lane - c_start[my]))
                                                : p.pool[c_off[my] + (pw + lane - c_start[my])];
                                const int last = __shfl_sync(0xffffffffu, my, 31);
                                src = last + (c_start[last + 1] == pw + 32 ? 1 : 0);
                                pw += 32;
                            }
                        }
#if LUSYM_MERGE_BATCH
                        // every window's visited word first (kU loads in flight, DSMEM in
                        // cluster mode), then the atomics on the bits that looked clear
                        uint32_t wv[kU];
#pragma unroll
                        for (int u = 0; u < kU; ++u)
                            wv[u] = jv[u] >= 0 ? *bm.word(jv[u] >> 5) : ~0u;
#endif
#pragma unroll
                        for (int u = 0; u < kU; ++u) {
                            const int j = jv[u];
#if LUSYM_MERGE_BATCH
                            const uint32_t bb = 1u << (j & 31);
                            const bool fr = j >= 0 && !(wv[u] & bb) &&
                                            !(atomicOr(bm.word(j >> 5), bb) & bb) && j < i;
#else
                            const bool fr = j >= 0 && bm.tas(j) && j < i;
#endif
                            if constexpr (CL && LUSYM_MERGE_HASH)
                                q_push_hashed<MODE>(fr, j, &h.cnt[nxt], nq,
                                                    gnq - (int64_t)bm.rank * 2 * p.spill_cap,
                                                    2 * p.spill_cap, bm.rank, bm.g, p.q);
                            else
                                q_push(fr, j, &h.cnt[nxt], nq, gnq, p.q);
                        }
                    }
                }
                __syncthreads();
#if LUSYM_MERGE_PROF
                if (tid == 0) {
                    prof_expand += clock64() - c_t1;
                    ++prof_tiles;
                    prof_entries += E;
                }
#endif
            }
            // (fsize > 0: the loop's barriers ordered every read of h.cnt[cur] before this)
            if (tid == 0 && fsize) h.cnt[cur] = 0;
            if (tid == 0) ++n_rounds;
#if LUSYM_MERGE_PROF
            ++rows_r;
#endif
            __syncthreads();
            cur = nxt;
        }
        // ---- output: the set bits, ascending, into the pool; publish the row.  Each rank
        // writes its own word slice at the offset of the slices before it.
        if (!fail) {
            if (tid == 0 && !diag && (i >> 5) >= bm.lo && (i >> 5) < bm.hi)
                atomicAnd(lw + (i >> 5), ~(1u << (i & 31)));
            __syncthreads();
            long long c = 0, lo = 0;
            for (int w = bm.lo + tid; w < bm.hi; w += NT) {
                const uint32_t x = lw[w];
                const int pc = __popc(x);
                c += pc;
                if (w < (i >> 5)) lo += pc;
                else if (w == (i >> 5)) lo += __popc(x & ((i & 31) == 31 ? 0xffffffffu
                                                                           : ((2u << (i & 31)) - 1u)));
            }
            block_sum2(c, lo, h);
            long long before = 0;
            if constexpr (CL) {
                if (tid == 0) {
                    h.part_c = c;
                    h.part_lo = lo;
                }
                cg::this_cluster().sync();
                long long tc = 0, tl = 0;
                for (int r = 0; r < bm.g; ++r) {
                    const MHdr *o = cg::this_cluster().map_shared_rank(&h, r);
                    if (r < bm.rank) before += o->part_c;
                    tc += o->part_c;
                    tl += o->part_lo;
                }
                c = tc;
                lo = tl;
            }
            if (tid == 0 && bm.rank == 0) {
                const unsigned long long o = atomicAdd(p.pool_cursor, (unsigned long long)c);
                const bool fits = o + (unsigned long long)c <= (unsigned long long)p.pool_cap;
                h.off = fits ? (long long)o : -1ll;
                if (fits) {
                    p.fill_count[i] = (int32_t)c;
                    p.ucut[i] = (int32_t)lo;
                }
            }
            csync_impl(CL);
            long long off = h.off;
            if constexpr (CL) off = cg::this_cluster().map_shared_rank(&h, 0)->off;
            if (off < 0) {
                fail = 1;
            } else {
                int32_t *dst = p.pool + off + before;
                long long run = 0;
                for (int w0 = bm.lo; w0 < bm.hi; w0 += NT) {
                    const int w = w0 + tid;
                    uint32_t x = w < bm.hi ? lw[w] : 0u;
                    long long tot;
                    long long pos = run + scan_excl(__popc(x), h, &tot);
                    for (; x; x &= x - 1, ++pos) dst[pos] = (w << 5) + __ffs(x) - 1;
                    run += tot;
                }
                __threadfence();
                csync_impl(CL);
                if (tid == 0 && bm.rank == 0) st_release(p.row_off + i, off);
            }
        }
        if (fail && tid == 0 && bm.rank == 0) {
            p.fail_list[atomicAdd(p.fail_cnt, 1ull)] = i;
            st_release(p.row_off + i, -1);
        }
#if LUSYM_MERGE_PROF
        if (tid == 0 && bm.rank == 0) {
            unsigned long long t_end;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
            printf("k_merge_rows: row %d cta %d claim %llu first_wait %+lld last_wait %+lld end %+lld "
                   "(ns after claim) rounds %llu waits %llu\n", i, (int)blockIdx.x, t_claim % 1000000000ull,
                   t_firstwait ? (long long)(t_firstwait - t_claim) : -1ll,
                   t_lastwait ? (long long)(t_lastwait - t_claim) : -1ll,
                   (long long)(t_end - t_claim), rows_r, nwaits_r);
            printf("k_merge_rows: row %d rank0 tiles %lld entries %lld setup cycles %lld expand "
                   "cycles %lld\n", i, prof_tiles, prof_entries, prof_setup, prof_expand);
        }
#endif
        // ---- fill(:) = 0 for the next row (L115)
        __syncthreads();
        for (int w = bm.lo + tid; w < bm.hi; w += NT) lw[w] = 0;
        if constexpr (CL)
            for (int w = tid; w < p.cl_filter; w += NT) bm.filt[w] = 0;
        // (the next claim's cluster barrier orders this before any rank's next seed)
    }
    if (tid == 0 && p.stats) {
        atomicAdd(p.stats + 0, n_read);
        atomicAdd(p.stats + 1, bm.rank == 0 ? n_rounds : 0ull);
        atomicAdd(p.stats + 2, n_waits);
    }
}

// ---- grid-wide mode (k_merge_grid): when only a few rows were deferred (cfg3: its 32 hubs),
// the clusters above finish them one after another anyway (each hub's closure contains the
// hubs below it), each on 4 SMs.  Here the whole grid takes the rows one at a time, in
// increasing order, so every deferred row below i is finished before i starts and nothing
// waits: the frontier's U segments are read by every SM (the step is a stream of pool reads)
// and test-and-set goes to one visited bitmap in HBM (L2-resident, n bits).  Grid barriers
// separate the phases: seed, then per round (lengths -> compaction -> expansion), then the
// output (popcounts -> pool offset -> sorted write).

// Test-and-set in the grid's visited bitmap (HBM, L2-resident) behind a per-CTA filter in
// shared memory (fw words, 0: none): bits are only ever set
// during a row, so a bit this CTA has seen set (in the filter) is set; a miss reads the global
// word and keeps every bit it holds.  Nearly every pool entry of a hub's closure is a member
// already found (cfg3: 1.3e9 entries read for 2.7e7 members), so most tests end in shared memory.
__device__ __forceinline__ bool tas_f(uint32_t *bits, uint32_t *filt, bool use, int v)
{
    const uint32_t b = 1u << (v & 31);
    const int w = v >> 5;
    if (use && (filt[w] & b)) return false;
    const uint32_t g = __ldcg(bits + w);
    bool fresh = false;
    uint32_t now = g;
    if (!(g & b)) {
        const uint32_t old = atomicOr(bits + w, b);
        fresh = !(old & b);
        now = old | b;
    }
    if (use) atomicOr(filt + w, now);
    return fresh;
}

// warp-aggregated append to a global frontier list
__device__ __forceinline__ void gpush(bool pred, int32_t v, int32_t *cnt, int32_t *list)
{
    const unsigned b = __ballot_sync(0xffffffffu, pred);
    if (!b) return;
    const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(cnt, __popc(b));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (pred) list[base + __popc(b & ((1u << lane) - 1u))] = v;
}

__device__ __forceinline__ int ld_cg_int(const int32_t *p) { return __ldcg(p); }

// new frontier members of this CTA, collected in shared memory and appended to the global
// list with one atomic per CTA per phase (a single global counter hit by every warp of the
// grid serialises at its L2 slice); past kGBuf entries a warp appends directly
constexpr int kGBuf = 4096;
struct GBuf {
    int32_t v[kGBuf];
    int cnt, base;
};
// segments staged for the expansion (starts with kSent look-ahead entries, pool offsets)
constexpr int kGSeg = 1024;
struct GSeg {
    long long st[kGSeg + kSent];
    long long off[kGSeg + kSent];
    int m;
};

__device__ __forceinline__ void gbuf_push(bool pred, int32_t v, GBuf &sb, int32_t *cnt,
                                          int32_t *list)
{
    const unsigned b = __ballot_sync(0xffffffffu, pred);
    if (!b) return;
    const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(&sb.cnt, __popc(b));
    base = __shfl_sync(0xffffffffu, base, leader);
    const int slot = base + __popc(b & ((1u << lane) - 1u));
    if (pred && slot < kGBuf) sb.v[slot] = v;
    gpush(pred && slot >= kGBuf, v, cnt, list);  // the part past the buffer, directly
}

// append the CTA's collected members to the global list (block-uniform; ends with a barrier)
__device__ __forceinline__ void gbuf_flush(GBuf &sb, int32_t *cnt, int32_t *list)
{
    __syncthreads();
    const int m = min(sb.cnt, kGBuf);
    if (threadIdx.x == 0) sb.base = m ? atomicAdd(cnt, m) : 0;
    __syncthreads();
    for (int k = threadIdx.x; k < m; k += NT) list[sb.base + k] = sb.v[k];
    __syncthreads();
    if (threadIdx.x == 0) sb.cnt = 0;
    __syncthreads();
}

__global__ void __launch_bounds__(NT, 1) k_merge_grid(const MergeParams p)
{
    cg::grid_group grid = cg::this_grid();
    __shared__ MHdr h;
    __shared__ GBuf sb;
    __shared__ GSeg sg;
    extern __shared__ uint32_t filt[];  // p.grid_filter words (0: no filter)
    const int tid = threadIdx.x, wid = tid >> 5, lane = tid & 31;
    const bool use_f = p.grid_filter > 0;
    if (tid == 0) sb.cnt = 0;
    for (int w = tid; w < p.grid_filter; w += NT) filt[w] = 0;
    __syncthreads();
    const int G = gridDim.x, b = blockIdx.x;
    const int nall = (int)min(*p.list_cnt, (unsigned long long)p.list_max);
    // all rows of a short list, or (grid_head) the first rows of any list: the head of the
    // hubs' dependency chain, whose closure is the tail's critical path on a cluster
    int nlist = nall <= p.grid_max ? nall : 0;
    if (p.grid_head > 0) nlist = min(nall, max(nlist, p.grid_head));
    if (nlist == 0) return;  // uniform: the cluster kernel takes them
    const int n = p.n, nw = (n + 31) >> 5;
    uint32_t *bits = p.gbits;  // zero on entry; every row clears what it set
    int32_t *ctrl = p.gctrl;   // [0], [1]: frontier counters; [2]: fail; [3]: diagonal
    long long *part = p.gpart;
    unsigned long long n_read = 0, n_rounds = 0;
#if LUSYM_MERGE_PROF  // diagnostic build: ns per phase (CTA 0's view), printed at the end
    unsigned long long tp[6] = {0, 0, 0, 0, 0, 0}, tq = 0;
#define MPROF(k)                                                                 \
    do {                                                                         \
        unsigned long long now_;                                                 \
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now_));                 \
        if (tq) tp[k] += now_ - tq;                                              \
        tq = now_;                                                               \
    } while (0)
#else
#define MPROF(k) do { } while (0)
#endif
    for (int r = 0; r < nlist; ++r) {
        const int i = p.list[r];
        MPROF(5);
        if (b == 0 && tid == 0) ctrl[0] = ctrl[1] = ctrl[2] = ctrl[3] = 0;
        grid.sync();  // (also orders the previous row's bitmap clears before this row's marks)
        if (b == 0 && tid == 0) atomicOr(bits + (i >> 5), 1u << (i & 31));
        // ---- seed: S = A(i,:); members t < i form the first frontier
        {
            const int64_t rb = p.rp[i], re = p.rp[i + 1];
            for (int64_t e0 = rb + (int64_t)b * NT; e0 < re; e0 += (int64_t)G * NT) {
                const int64_t e = e0 + tid;
                bool fr = false;
                int v = -1;
                if (e < re) {
                    v = __ldg(p.ci + e);
                    if (v == i) ctrl[3] = 1;
                    else fr = tas_f(bits, filt, use_f, v) && v < i;
                }
                gbuf_push(fr, v, sb, ctrl + 0, p.gq);
            }
            gbuf_flush(sb, ctrl + 0, p.gq);
        }
        grid.sync();
        MPROF(0);
        int cur = 0;
        for (;;) {
            // (the fail flag is only read right after the barrier that follows its writes:
            // every CTA must take the same branches around grid.sync)
            const int fsize = ld_cg_int(ctrl + cur);
            if (fsize == 0) break;
            const int nxt = cur ^ 1;
            const int32_t *F = p.gq + (size_t)cur * n;
            int32_t *NF = p.gq + (size_t)nxt * n;
            // (a) each member's U segment (pool offset, length); per-CTA sums over a
            //     contiguous chunk of members: total length and non-empty segments
            const int chunk = (fsize + G - 1) / G;
            const int k0 = min(fsize, b * chunk), k1 = min(fsize, k0 + chunk);
            long long sl = 0, sn = 0;
            for (int k = k0 + tid; k < k1; k += NT) {
                const int t = __ldcg(F + k);
                const int64_t o = ld_acquire(p.row_off + t);
                long long len = 0, off = 0;
                if (o < 0) {
                    ctrl[2] = 1;  // row t is not in the pool (unstaged, or failed)
                } else {
                    const int uc = __ldcg(p.ucut + t);
                    off = o + uc;
                    len = (long long)__ldcg(p.fill_count + t) - uc;
                }
                p.glen[k] = len;
                p.goff[k] = off;
                sl += len;
                sn += len > 0;
            }
            block_sum2(sl, sn, h);
            if (tid == 0) {
                part[b] = sl;
                part[G + b] = sn;
            }
            if (b == 0 && tid == 0) ctrl[nxt] = 0;  // last read as a fsize two barriers ago
            grid.sync();
            MPROF(1);
            if (ld_cg_int(ctrl + 2)) break;
            // (b) compaction of the non-empty segments, in member order
            long long bl = 0, bn = 0, E = 0, M = 0;
            for (int c = tid; c < G; c += NT) {
                const long long x = __ldcg(part + c), y = __ldcg(part + G + c);
                E += x;
                M += y;
                if (c < b) {
                    bl += x;
                    bn += y;
                }
            }
            block_sum2(bl, bn, h);
            block_sum2(E, M, h);
            for (int kb = k0; kb < k1; kb += NT) {
                const int k = kb + tid;
                long long len = 0;
                if (k < k1) len = __ldcg(p.glen + k);
                long long tot;
                // (len << 20 | nonempty): chunk <= ceil(n / G) members, so counts fit 20 bits
                const long long st = scan_excl((len << 20) | (len > 0 ? 1 : 0), h, &tot);
                if (len > 0) {
                    const long long m = bn + (st & 0xfffff);
                    p.gstart[m] = bl + (st >> 20);
                    p.gcoff[m] = __ldcg(p.goff + k);
                }
                bl += tot >> 20;
                bn += tot & 0xfffff;
            }
            if (b == 0 && tid < kSent) p.gstart[M + tid] = LLONG_MAX;
            if (b == 0 && tid == 0) n_read += (unsigned long long)E;
            grid.sync();
            MPROF(2);
            // (c) expansion: CTA b takes the flat positions [b per, (b+1) per); the starts and
            //     offsets of the segments they cover are staged in shared memory kGSeg at a
            //     time, then each warp expands a contiguous chunk as k_merge_rows does (one
            //     search, then 32 start bits per window, all in shared memory)
            {
                const long long per = ((E + G - 1) / G + 31) & ~31ll;
                const long long fb = min(E, (long long)b * per), fe = min(E, fb + per);
                if (fb < fe) {
                    if (tid == 0) {
                        int lo = 0, hi = (int)M - 1;  // last segment starting at or before fb
                        while (lo < hi) {
                            const int mid = (lo + hi + 1) >> 1;
                            if (__ldcg(p.gstart + mid) <= fb) lo = mid; else hi = mid - 1;
                        }
                        sg.m = lo;
                    }
                    __syncthreads();
                    int m = sg.m;
                    long long pos = fb;
                    while (pos < fe) {
                        for (int k = tid; k < kGSeg + kSent; k += NT) {
                            const long long mk = (long long)m + k;
                            sg.st[k] = mk < M + kSent ? __ldcg(p.gstart + mk) : LLONG_MAX;
                            sg.off[k] = mk < M ? __ldcg(p.gcoff + mk) : 0;
                        }
                        __syncthreads();
                        const long long bend = min(fe, sg.st[kGSeg]);
                        const long long C = ((bend - pos + NW - 1) / NW + 31) & ~31ll;
                        long long pw = pos + (long long)wid * C;
                        const long long pend = min(bend, pw + C);
                        if (pw < pend) {
                            int src = 0;
#pragma unroll
                            for (int step = kGSeg / 2; step >= 1; step >>= 1)
                                if (src + step < kGSeg && sg.st[src + step] <= pw) src += step;
                            while (pw < pend) {
                                int jv[kU];
#pragma unroll
                                for (int u = 0; u < kU; ++u) {
                                    jv[u] = -1;
                                    if (pw < pend) {
                                        const long long snx = sg.st[src + 1 + lane];
                                        const unsigned bit =
                                            snx < pw + 32 ? 1u << (int)(snx - pw) : 0u;
                                        const unsigned mask = __reduce_or_sync(0xffffffffu, bit);
                                        const int my = src + __popc(mask & ((2u << lane) - 1u));
                                        if (pw + lane < pend)
                                            jv[u] = p.pool[sg.off[my] + (pw + lane - sg.st[my])];
                                        const int last = __shfl_sync(0xffffffffu, my, 31);
                                        src = last + (sg.st[last + 1] == pw + 32 ? 1 : 0);
                                        pw += 32;
                                    }
                                }
#pragma unroll
                                for (int u = 0; u < kU; ++u) {
                                    const int j = jv[u];
                                    const bool fr = j >= 0 && tas_f(bits, filt, use_f, j) && j < i;
                                    gbuf_push(fr, j, sb, ctrl + nxt, NF);
                                }
                            }
                        }
                        __syncthreads();
                        pos = bend;
                        m += kGSeg;
                    }
                }
            }
            gbuf_flush(sb, ctrl + nxt, NF);
            ++n_rounds;
            grid.sync();
            MPROF(3);
            cur = nxt;
        }
        const bool fail = ld_cg_int(ctrl + 2) != 0;
        const bool diag = ld_cg_int(ctrl + 3) != 0;
        // ---- output: the set bits, ascending, into the pool (each CTA a contiguous run of
        // words at the offset of the runs before it); publish the row
        const int wchunk = (nw + G - 1) / G;
        const int w0 = min(nw, b * wchunk), w1 = min(nw, w0 + wchunk);
        if (!fail) {
            if (!diag && tid == 0 && (i >> 5) >= w0 && (i >> 5) < w1)
                atomicAnd(bits + (i >> 5), ~(1u << (i & 31)));
            __syncthreads();
            long long c = 0, lo = 0;
            for (int w = w0 + tid; w < w1; w += NT) {
                const uint32_t x = __ldcg(bits + w);
                const int pc = __popc(x);
                c += pc;
                if (w < (i >> 5)) lo += pc;
                else if (w == (i >> 5))
                    lo += __popc(x & ((i & 31) == 31 ? 0xffffffffu : ((2u << (i & 31)) - 1u)));
            }
            block_sum2(c, lo, h);
            if (tid == 0) {
                part[2 * G + b] = c;
                part[3 * G + b] = lo;
            }
            grid.sync();
            long long before = 0, tc = 0, tl = 0, dummy = 0;
            for (int q = tid; q < G; q += NT) {
                const long long x = __ldcg(part + 2 * G + q);
                tc += x;
                tl += __ldcg(part + 3 * G + q);
                if (q < b) before += x;
            }
            block_sum2(before, dummy, h);
            block_sum2(tc, tl, h);
            if (b == 0 && tid == 0) {
                const unsigned long long o = atomicAdd(p.pool_cursor, (unsigned long long)tc);
                const bool fits = o + (unsigned long long)tc <= (unsigned long long)p.pool_cap;
                part[4 * G] = fits ? (long long)o : -1ll;
                if (fits) {
                    p.fill_count[i] = (int32_t)tc;
                    p.ucut[i] = (int32_t)tl;
                } else {
                    ctrl[2] = 1;
                }
            }
            grid.sync();
            const long long off = __ldcg(part + 4 * G);
            if (off >= 0) {
                int32_t *dst = p.pool + off + before;
                long long run = 0;
                for (int wb = w0; wb < w1; wb += NT) {
                    const int w = wb + tid;
                    uint32_t x = w < w1 ? __ldcg(bits + w) : 0u;
                    long long tot;
                    long long pos = run + scan_excl(__popc(x), h, &tot);
                    for (; x; x &= x - 1, ++pos) dst[pos] = (w << 5) + __ffs(x) - 1;
                    run += tot;
                }
                __threadfence();
            }
        }
        grid.sync();  // every CTA's pool writes (and reads of the bitmap) are done
        if (b == 0 && tid == 0) {
            const long long off = fail ? -1ll : __ldcg(part + 4 * G);
            if (off >= 0) {
                st_release(p.row_off + i, off);
            } else {
                p.fail_list[atomicAdd(p.fail_cnt, 1ull)] = i;
                st_release(p.row_off + i, -1);
            }
        }
        // fill(:) = 0 for the next row (L115): each CTA its own words, and its whole filter
        for (int w = w0 + tid; w < w1; w += NT) bits[w] = 0;
        for (int w = tid; w < p.grid_filter; w += NT) filt[w] = 0;
        MPROF(4);
        // (the next row's first barrier orders this before its seed)
    }
#if LUSYM_MERGE_PROF
    if (b == 0 && tid == 0)
        printf("k_merge_grid: rows %d rounds %llu read %llu | ns seed %llu lens %llu compact %llu "
               "expand %llu output %llu other %llu\n", nlist, n_rounds, n_read, tp[0], tp[1],
               tp[2], tp[3], tp[4], tp[5]);
#endif
    if (b == 0 && tid == 0) {
        *p.counter = (unsigned long long)nlist;  // the cluster kernel after this claims nothing
        if (p.stats) {
            atomicAdd(p.stats + 0, n_read);
            atomicAdd(p.stats + 1, n_rounds);
        }
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

// ---- row sharding with deferred rows (LU_F_DEFER_GLOBAL)
__global__ void k_list_to_flags(const int32_t *list, const unsigned long long *cnt, int32_t max,
                                int32_t *flags, int32_t *fill_count, int32_t value)
{
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= (int)min(*cnt, (unsigned long long)max)) return;
    if (flags) flags[list[k]] = value;
    if (fill_count) fill_count[list[k]] = 0;
}

// the assembled CSR as the tail's pool: row_off = row_ptr (kRowDeferred for flagged rows),
// ucut = entries <= i of row i (binary search in the sorted row)
__global__ void k_prep_merge(int32_t n, const int32_t *flags, const int64_t *rp, const int32_t *ci,
                             int64_t *row_off, int32_t *ucut)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    if (flags[i]) {
        row_off[i] = kRowDeferred;
        return;
    }
    int64_t lo = rp[i], hi = rp[i + 1];
    const int64_t b = lo;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (ci[mid] <= i) lo = mid + 1; else hi = mid;
    }
    row_off[i] = b;
    ucut[i] = (int32_t)(lo - b);
}

__global__ void k_scatter_flagged(int32_t n, const int32_t *flags, const int64_t *pos,
                                  int32_t *list)
{
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n && flags[i]) list[pos[i]] = i;
}

int cluster_shift(int n, int g)
{
    const int nw = (n + 31) / 32;
    const int per = (nw + g - 1) / g;
    int sh = 0;
    while ((1 << sh) < per) ++sh;
    return sh;
}

}  // namespace

size_t merge_grid_smem(int n, int *filter_words)
{
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaFuncAttributes fa;
    if (cudaFuncGetAttributes(&fa, k_merge_grid) != cudaSuccess) {
        cudaGetLastError();
        *filter_words = 0;
        return 0;
    }
    const size_t fw = (size_t)(n + 31) / 32;
    const bool fits = fa.sharedSizeBytes + fw * 4 <= (size_t)optin &&
                      !getenv("LUSYM_MERGE_GRID_NOFILTER");  // A/B knob
    *filter_words = fits ? (int)fw : 0;
    return fits ? fw * 4 : 0;
}

cudaError_t merge_grid_size(int n, int *grid, int *filter_words)
{
    int dev = 0, sms = 0, occ = 0;
    cudaGetDevice(&dev);
    const size_t smem = merge_grid_smem(n, filter_words);
    cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute((const void *)k_merge_grid,
                                 cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_merge_grid, NT, smem);
    if (e != cudaSuccess) return e;
    *grid = sms * (occ > 0 ? occ : 0);
    return cudaSuccess;
}

cudaError_t merge_grid_launch(const MergeParams &p, int grid, cudaStream_t s)
{
    void *args[] = {(void *)&p};
    return cudaLaunchCooperativeKernel((const void *)k_merge_grid, grid, NT, args,
                                       (size_t)p.grid_filter * 4, s);
}

cudaError_t merge_configure_impl(size_t smem);
cudaError_t merge_max_clusters_impl(int g, size_t smem, int *clusters);

size_t merge_smem_bytes(int n, int mode, int g, int q, bool filter)
{
    size_t b = kHdrBytes + (2 * (size_t)NT + kSent) * sizeof(long long) +
               2 * (size_t)q * sizeof(int32_t);
    if (mode == 0) b += (size_t)((n + 31) / 32) * sizeof(uint32_t);
    if (mode == 2) b += ((size_t)1 << cluster_shift(n, g)) * sizeof(uint32_t);
    if (mode == 2 && filter) b += (size_t)((n + 31) / 32) * sizeof(uint32_t);
    return (b + 15) & ~(size_t)15;
}

cudaError_t merge_configure(size_t smem)
{
    static size_t done[64];  // per device: the largest size already set
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && done[dev] >= smem) return cudaSuccess;
    cudaError_t e0 = merge_configure_impl(smem);
    if (e0 == cudaSuccess && dev >= 0 && dev < 64) done[dev] = smem;
    return e0;
}

cudaError_t merge_configure_impl(size_t smem)
{
    const void *fns[3] = {(const void *)k_merge_rows<0>, (const void *)k_merge_rows<1>,
                          (const void *)k_merge_rows<2>};
    for (const void *f : fns) {
        cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
    }
    return cudaFuncSetAttribute((const void *)k_merge_rows<2>,
                                cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
}

cudaError_t merge_max_clusters(int g, size_t smem, int *clusters)
{
    static std::map<std::tuple<int, int, size_t>, int> cache;
    static std::mutex mu;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    const auto key = std::make_tuple(dev, g, smem);
    auto it = cache.find(key);
    if (it != cache.end()) {
        *clusters = it->second;
        return cudaSuccess;
    }
    cudaError_t e0 = merge_max_clusters_impl(g, smem, clusters);
    if (e0 == cudaSuccess) cache[key] = *clusters;
    return e0;
}

cudaError_t merge_max_clusters_impl(int g, size_t smem, int *clusters)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(g * 64, 1, 1);
    cfg.blockDim = dim3(NT, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = g;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaOccupancyMaxActiveClusters(clusters, (const void *)k_merge_rows<2>, &cfg);
}

cudaError_t zero_deferred_counts(const int32_t *list, const unsigned long long *cnt, int32_t max,
                                 int32_t *fill_count, cudaStream_t s)
{
    k_list_to_flags<<<(max + 255) / 256, 256, 0, s>>>(list, cnt, max, nullptr, fill_count, 0);
    return cudaGetLastError();
}

cudaError_t deferred_to_flags(const int32_t *list, const unsigned long long *cnt, int32_t max,
                              int32_t *flags, cudaStream_t s)
{
    k_list_to_flags<<<(max + 255) / 256, 256, 0, s>>>(list, cnt, max, flags, nullptr, 1);
    return cudaGetLastError();
}

cudaError_t prep_merge(int32_t n, const int32_t *flags, const int64_t *rp, const int32_t *ci,
                       int64_t *row_off, int32_t *ucut, const int64_t *flag_pos, int32_t *list,
                       cudaStream_t s)
{
    if (n <= 0) return cudaSuccess;
    k_prep_merge<<<(n + 255) / 256, 256, 0, s>>>(n, flags, rp, ci, row_off, ucut);
    k_scatter_flagged<<<(n + 255) / 256, 256, 0, s>>>(n, flags, flag_pos, list);
    return cudaGetLastError();
}

cudaError_t merge_sort_list(int32_t *list, const unsigned long long *cnt, int32_t max,
                            cudaStream_t s)
{
    k_sort_list<<<1, 1024, 0, s>>>(list, cnt, max);
    return cudaGetLastError();
}

cudaError_t merge_launch(const MergeParams &p, int mode, int g, int grid, size_t smem,
                         cudaStream_t s)
{
    static_assert(sizeof(MHdr) <= kHdrBytes, "merge header too large");
    if (mode == 0) {
        k_merge_rows<0><<<grid, NT, smem, s>>>(p, 0);
    } else if (mode == 1) {
        k_merge_rows<1><<<grid, NT, smem, s>>>(p, 0);
    } else {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid, 1, 1);  // CTAs: a multiple of g
        cfg.blockDim = dim3(NT, 1, 1);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = g;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        const int sh = cluster_shift(p.n, g);
        return cudaLaunchKernelEx(&cfg, k_merge_rows<2>, p, sh);
    }
    return cudaGetLastError();
}

}  // namespace lusym
