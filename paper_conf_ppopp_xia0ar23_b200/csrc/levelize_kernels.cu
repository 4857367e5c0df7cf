// Levelization (S8 + S9): Algorithm 5 of PAPER.md (L290-320) on sm_100a.
//
//   cons_graph   (L308): the dependency graph is a VIEW of the L+U CSR: the successors of
//                column i are the strict-U entries of row i (rule "U(i,j)!=0 => j depends on
//                i", L167), pruned to the prefix up to the first symmetric pair
//                p_i = min{k > i : (i,k),(k,i) in P}, which is exact for longest paths
//                (reading R27); the GLU3 reading (R12) adds the transpose of strict L.
//                Chains u -> v with outdeg(u) = 1 = indeg(v) are then contracted (list ranking
//                by pointer jumping): along a chain level(v) = level(head) + rank(v), so Kahn
//                only has to order chain heads.  Both reductions preserve every level exactly;
//                LU_F_NO_PRUNE / LU_F_NO_CONTRACT switch them off (plain Alg. 5).
//   cnt_indegree (L311): atomic histogram over the successor lists.
//   Topo         (L293-306): ONE persistent cooperative kernel replaces the parent kernel and
//                its dynamically launched children (device-side cudaDeviceSynchronize is gone
//                on sm_90+).  Wide rounds: every CTA relaxes the queue (warp per queued chain,
//                lanes over its tail's successors), grid barrier per round.  Narrow rounds
//                (queue <= kNarrowMax): CTA 0 alone runs round after round with a shared-memory
//                queue and __syncthreads while the other CTAs wait at the next grid barrier.
//   level(k) = max(-1, level(preds)) + 1 (L283): a head's level is the max over its
//   predecessor chains of (their head level + length), final when its in-degree reaches 0;
//   each head is enqueued exactly once, on that decrement (reading R14).
#include "internal.h"

#include <cooperative_groups.h>

#include <climits>

namespace cg = cooperative_groups;

namespace lusym {
namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kKahnNT = 512;
constexpr int kNarrowQ = 4096;   // shared queue entries per buffer (narrow phase)
constexpr int kNarrowMax = 2048; // queue size at or below which CTA 0 runs alone

// ctrl block layout (int32)
enum {
    kQ0 = 0, kQ1 = 1, kQ2 = 2, kRound = 3, kWide = 4, kNarrow = 5, kMaxLevel = 6,
    kChanged = 8, /* 8..10 rotating flags of the list-ranking loop */ kCtrlInts = 16
};

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
// psym (GLU3 rule with pruning, else null): psym[i] = p_i, or INT_MAX without a symmetric pair.
__global__ void k_urange(int32_t n, const int64_t *rp, const int32_t *ci, int prune,
                         int64_t *ustart, int64_t *uend, int32_t *psym)
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
        bool sym = false;
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
                    sym = true;
                    break;
                }
            }
        }
        if (lane == 0) {
            ustart[i] = us;
            uend[i] = ue;
            if (psym) psym[i] = sym ? ci[ue - 1] : INT_MAX;
        }
    }
}

// GLU3 reading: count strict-L entries per column (transpose sizes).  With psym (pruning,
// reading R32) the entry (r, c) is kept only for r < p_c: a successor r > p_c of c is implied
// through p_c (the fill rule on (r,c),(c,p_c) gives (r,p_c)), and r = p_c is already c's U edge.
__global__ void k_lt_count(int32_t n, const int64_t *rp, const int32_t *ci,
                           const int64_t *ustart, const int32_t *psym, int32_t *cnt)
{
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = wg; r < n; r += nwarps) {
        const int64_t a = rp[r], b = ustart[r];
        for (int64_t k = a + lane; k < b; k += 32) {
            const int c = ci[k];
            if (c < r && (!psym || r < psym[c])) atomicAdd(cnt + c, 1);
        }
    }
}

__global__ void k_lt_fill(int32_t n, const int64_t *rp, const int32_t *ci, const int64_t *ustart,
                          const int32_t *psym, unsigned long long *cursor, int32_t *lt_idx)
{
    const int lane = threadIdx.x & 31;
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = wg; r < n; r += nwarps) {
        const int64_t a = rp[r], b = ustart[r];
        for (int64_t k = a + lane; k < b; k += 32) {
            const int c = ci[k];
            if (c < r && (!psym || r < psym[c])) lt_idx[atomicAdd(cursor + c, 1ull)] = (int)r;
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

// chain links: u -> v is a link iff u has exactly one successor v and v exactly one predecessor.
// J[v] = link predecessor (or v), D[v] = 1 for linked v (else 0), nxt[u] = v or -1.
__global__ void k_link(int32_t n, const int32_t *ci, const int64_t *us, const int64_t *ue,
                       const int64_t *ltp, const int32_t *lti, const int32_t *indeg, int contract,
                       int32_t *J, int32_t *D, int32_t *nxt)
{
    const int u = blockIdx.x * blockDim.x + threadIdx.x;
    if (u >= n) return;
    int v = -1;
    if (contract) {
        const int64_t du = ue[u] - us[u];
        const int64_t dl = ltp ? ltp[u + 1] - ltp[u] : 0;
        if (du + dl == 1) {
            const int c = du ? ci[us[u]] : lti[ltp[u]];
            if (indeg[c] == 1) v = c;
        }
    }
    nxt[u] = v;
    if (v >= 0) {
        J[v] = u;
        D[v] = 1;
    }
}

__global__ void k_link_init(int32_t n, int32_t *J, int32_t *D)
{
    const int v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v < n) {
        J[v] = v;
        D[v] = 0;
    }
}

// list ranking by pointer jumping: after the loop J[v] = chain head, D[v] = rank in the chain
__global__ void __launch_bounds__(256) k_rank(int32_t n, int32_t *J0, int32_t *D0, int32_t *J1,
                                              int32_t *D1, int32_t *ctrl, int32_t *rounds_out)
{
    cg::grid_group grid = cg::this_grid();
    int32_t *Ja = J0, *Da = D0, *Jb = J1, *Db = D1;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    int r = 0;
    for (;; ++r) {
        int32_t *flag = ctrl + kChanged + r % 3;
        if (t0 == 0) ctrl[kChanged + (r + 1) % 3] = 0;
        bool changed = false;
        for (int64_t v = t0; v < n; v += stride) {
            const int j = __ldcg(Ja + v);
            const int jj = __ldcg(Ja + j);
            Jb[v] = jj;
            Db[v] = __ldcg(Da + v) + (j != v ? __ldcg(Da + j) : 0);
            changed |= jj != j;
        }
        if (__syncthreads_or(changed) && threadIdx.x == 0) atomicOr(flag, 1);
        grid.sync();
        int32_t *t = Ja; Ja = Jb; Jb = t;
        t = Da; Da = Db; Db = t;
        if (__ldcg(flag) == 0) break;
    }
    // make sure the final result is in (J0, D0)
    if (Ja != J0) {
        for (int64_t v = t0; v < n; v += stride) {
            J0[v] = Ja[v];
            D0[v] = Da[v];
        }
    }
    if (t0 == 0) *rounds_out = r + 1;
}

// per chain: tail and length (stored at the head), and the tail's successor range, so that
// relaxing a head is one 16-byte load away from its successor list (no tail -> range chain)
__global__ void k_chain_info(int32_t n, const int32_t *J, const int32_t *D, const int32_t *nxt,
                             const int64_t *us, const int64_t *ue, int32_t *tail, int32_t *len,
                             longlong2 *hu)
{
    const int v = blockIdx.x * blockDim.x + threadIdx.x;
    if (v >= n) return;
    if (nxt[v] < 0) {
        const int h = J[v];
        tail[h] = v;
        len[h] = D[v] + 1;
        hu[h] = make_longlong2(us[v], ue[v]);
    }
}

// cons_queue for round 0 (L294-296): heads with in-degree 0
__global__ void k_init_queue(int32_t n, const int32_t *indeg, const int32_t *J, int32_t *best,
                             int32_t *q0, int32_t *ctrl)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    bool src = false;
    if (j < n) {
        best[j] = 0;
        src = J[j] == j && indeg[j] == 0;
    }
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
    const int32_t *tail, *len;
    const longlong2 *hu;  // [n] per head: successor range of its chain's tail
    int32_t *indeg, *best, *queue;  // queue: 2 x n
    int32_t *ctrl;
    int32_t narrow_max;
    int32_t wide_only;
};

__device__ __forceinline__ int ld_ctrl(const int32_t *p) { return __ldcg(p); }

// relax the successors v of chain h (update, L299 + cons_queue, L302, fused)
template <class Push>
__device__ __forceinline__ void relax(const KahnArgs &A, int h, Push &&push)
{
    const int lane = threadIdx.x & 31;
    const longlong2 r = A.hu[h];                    // the tail's successor range
    const int lvl = __ldcg(A.best + h) + A.len[h];  // level of every successor via this chain
    const int64_t a = r.x, b = r.y;
    for (int64_t eb = a; eb < b; eb += 32) {
        const int64_t e = eb + lane;
        bool z = false;
        int v = 0;
        if (e < b) {
            v = A.ci[e];
            atomicMax(A.best + v, lvl);
            z = atomicSub(A.indeg + v, 1) == 1;
        }
        push(z, v);
    }
    if (A.ltp) {
        const int t = A.tail[h];
        const int64_t c = A.ltp[t], d = A.ltp[t + 1];
        for (int64_t eb = c; eb < d; eb += 32) {
            const int64_t e = eb + lane;
            bool z = false;
            int v = 0;
            if (e < d) {
                v = A.lti[e];
                atomicMax(A.best + v, lvl);
                z = atomicSub(A.indeg + v, 1) == 1;
            }
            push(z, v);
        }
    }
}

__device__ __forceinline__ int warp_push_slot(bool pred, int *cnt)
{
    const unsigned b = __ballot_sync(kFull, pred);
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
    int L = 0;  // round number
    for (;;) {
        const int q = ld_ctrl(A.ctrl + L % 3);
        if (q == 0) break;
        int32_t *Q = A.queue + (size_t)(L & 1) * A.n;
        int32_t *NQ = A.queue + (size_t)((L + 1) & 1) * A.n;
        if (q <= A.narrow_max && !A.wide_only) {
            if (blockIdx.x == 0) {
                // ---- narrow phase: CTA 0 alone, shared queue, __syncthreads per round
                int32_t *cur = sq, *nxt = sq + kNarrowQ;
                for (int k = tid; k < q; k += kKahnNT) cur[k] = __ldcg(Q + k);
                if (tid == 0) scnt[0] = scnt[1] = scnt[2] = 0;
                __syncthreads();
                int qq = q, it = 0, lv = L, nq = 0;
                for (;;) {
                    int *cnt = &scnt[(it + 1) % 3];
                    if (tid == 0) scnt[(it + 2) % 3] = 0;
                    int32_t *gnext = A.queue + (size_t)((lv + 1) & 1) * A.n;
                    for (int k = warp; k < qq; k += NW) {
                        relax(A, cur[k], [&](bool z, int v) {
                            const int pos = warp_push_slot(z, cnt);
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
                    A.ctrl[kRound] = lv;
                    A.ctrl[kNarrow] += it;
                }
            }
            grid.sync();
            L = ld_ctrl(A.ctrl + kRound);
            continue;
        }
        // ---- wide round: all CTAs
        if (blockIdx.x == 0 && tid == 0) {
            A.ctrl[(L + 2) % 3] = 0;
            A.ctrl[kWide] += 1;
        }
        int *gcnt = A.ctrl + (L + 1) % 3;
        for (int k = gwarp; k < q; k += twarps) {
            relax(A, __ldcg(Q + k), [&](bool z, int v) {
                const int pos = warp_push_slot(z, gcnt);
                if (z) NQ[pos] = v;
            });
        }
        grid.sync();
        ++L;
    }
    if (blockIdx.x == 0 && tid == 0) A.ctrl[kRound] = L;
}

// level(v) = level(head) + rank(v); num_levels = max + 1
__global__ void k_expand(int32_t n, const int32_t *J, const int32_t *D, const int32_t *best,
                         int32_t *level, int32_t *ctrl)
{
    const int v = blockIdx.x * blockDim.x + threadIdx.x;
    int l = -1;
    if (v < n) {
        l = best[J[v]] + D[v];
        level[v] = l;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) l = max(l, __shfl_xor_sync(kFull, l, o));
    if ((threadIdx.x & 31) == 0) atomicMax(ctrl + kMaxLevel, l);
}

constexpr int kAuxNT = 256;

int aux_grid(int64_t warps)
{
    int64_t blocks = (warps * 32 + kAuxNT - 1) / kAuxNT;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (blocks < 1) blocks = 1;
    return (int)blocks;
}

}  // namespace

void levelize_free(LevelizeScratch &s, cudaStream_t st)
{
    dev_free(s.ustart, st); dev_free(s.uend, st); dev_free(s.indeg, st); dev_free(s.queue, st);
    dev_free(s.lt_ptr, st); dev_free(s.lt_idx, st); dev_free(s.lt_fill, st);
    dev_free(s.scan_blk, st); dev_free(s.ctrl, st); dev_free(s.chain, st);
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
                         bool prune, bool contract, bool wide_only, LevelizeScratch &s,
                         int32_t *level, LevelizeInfo *info, cudaStream_t st, const char **err)
{
    *info = LevelizeInfo();
    if (n == 0) return cudaSuccess;
    if (s.n_cap < n) {
        dev_free(s.ustart, st); dev_free(s.uend, st); dev_free(s.indeg, st);
        dev_free(s.queue, st); dev_free(s.lt_ptr, st); dev_free(s.lt_fill, st);
        dev_free(s.scan_blk, st); dev_free(s.ctrl, st); dev_free(s.chain, st);
        s.ustart = s.uend = s.lt_ptr = s.lt_fill = s.scan_blk = nullptr;
        s.indeg = s.queue = s.ctrl = s.chain = nullptr;
        LV_CK(dev_alloc((void **)&s.ustart, sizeof(int64_t) * n, st));
        LV_CK(dev_alloc((void **)&s.uend, sizeof(int64_t) * n, st));
        LV_CK(dev_alloc((void **)&s.indeg, sizeof(int32_t) * n, st));
        LV_CK(dev_alloc((void **)&s.queue, sizeof(int32_t) * 2 * (size_t)n, st));
        LV_CK(dev_alloc((void **)&s.lt_ptr, sizeof(int64_t) * ((size_t)n + 1), st));
        LV_CK(dev_alloc((void **)&s.lt_fill, sizeof(int64_t) * n, st));
        LV_CK(dev_alloc((void **)&s.scan_blk, sizeof(int64_t) * scan_scratch_elems(n), st));
        LV_CK(dev_alloc((void **)&s.ctrl, sizeof(int32_t) * kCtrlInts, st));
        LV_CK(dev_alloc((void **)&s.chain, sizeof(int32_t) * 12 * (size_t)n, st));
        s.n_cap = n;
    }
    int32_t *J0 = s.chain, *D0 = J0 + n, *J1 = D0 + n, *D1 = J1 + n, *nxt = D1 + n;
    int32_t *tail = nxt + n, *len = tail + n, *best = len + n;
    longlong2 *hu = reinterpret_cast<longlong2 *>(best + n);  // 16 n bytes, 16-B aligned
    const bool glu3 = rule == 1;
    const int g = aux_grid(n);
    const int gt = (n + 255) / 256;
    // cons_graph: strict-U ranges (pruned for the U rule)
    // psym lives in `best` until k_init_queue writes it
    int32_t *psym = (prune && glu3) ? best : nullptr;
    k_urange<<<g, kAuxNT, 0, st>>>(n, rp_lu, ci_lu, prune ? 1 : 0, s.ustart, s.uend, psym);
    LV_CK(cudaGetLastError());
    info->launches = 1;
    const int64_t *ltp = nullptr;
    const int32_t *lti = nullptr;
    if (glu3) {
        int32_t *cnt = s.indeg;  // reuse as a temporary int32[n]
        LV_CK(cudaMemsetAsync(cnt, 0, sizeof(int32_t) * n, st));
        k_lt_count<<<g, kAuxNT, 0, st>>>(n, rp_lu, ci_lu, s.ustart, psym, cnt);
        LV_CK(cudaGetLastError());
        LV_CK(scan_counts(n, cnt, s.lt_ptr, s.scan_blk, st));
        int64_t nl = 0;
        LV_CK(cudaMemcpyAsync(&nl, s.lt_ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        LV_CK(cudaStreamSynchronize(st));
        if (s.lt_cap < nl || s.lt_idx == nullptr) {
            dev_free(s.lt_idx, st);
            s.lt_idx = nullptr;
            LV_CK(dev_alloc((void **)&s.lt_idx, sizeof(int32_t) * (size_t)(nl > 0 ? nl : 1), st));
            s.lt_cap = nl;
        }
        LV_CK(cudaMemcpyAsync(s.lt_fill, s.lt_ptr, sizeof(int64_t) * n, cudaMemcpyDeviceToDevice,
                              st));
        k_lt_fill<<<g, kAuxNT, 0, st>>>(n, rp_lu, ci_lu, s.ustart, psym,
                                        reinterpret_cast<unsigned long long *>(s.lt_fill),
                                        s.lt_idx);
        LV_CK(cudaGetLastError());
        ltp = s.lt_ptr;
        lti = s.lt_idx;
        info->launches += 5;
    }
    // cnt_indegree
    LV_CK(cudaMemsetAsync(s.indeg, 0, sizeof(int32_t) * n, st));
    k_indeg<<<g, kAuxNT, 0, st>>>(n, ci_lu, s.ustart, s.uend, ltp, lti, s.indeg);
    LV_CK(cudaGetLastError());
    // chain contraction (list ranking)
    LV_CK(cudaMemsetAsync(s.ctrl, 0, sizeof(int32_t) * kCtrlInts, st));
    k_link_init<<<gt, 256, 0, st>>>(n, J0, D0);
    LV_CK(cudaGetLastError());
    k_link<<<gt, 256, 0, st>>>(n, ci_lu, s.ustart, s.uend, ltp, lti, s.indeg, contract ? 1 : 0,
                               J0, D0, nxt);
    LV_CK(cudaGetLastError());
    info->launches += 3;
    int dev = 0, sms = 0;
    LV_CK(cudaGetDevice(&dev));
    LV_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    if (contract) {
        int occ = 0;
        LV_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_rank, 256, 0));
        int grid = sms * (occ < 4 ? occ : 4);
        int32_t *rounds_dev = s.ctrl + 12;
        int32_t nn = n;
        void *args[] = {&nn, &J0, &D0, &J1, &D1, &s.ctrl, &rounds_dev};
        LV_CK(cudaLaunchCooperativeKernel((const void *)k_rank, grid, 256, args, 0, st));
        info->launches += 1;
    }
    k_chain_info<<<gt, 256, 0, st>>>(n, J0, D0, nxt, s.ustart, s.uend, tail, len, hu);
    LV_CK(cudaGetLastError());
    // cons_queue (round 0)
    k_init_queue<<<gt, 256, 0, st>>>(n, s.indeg, J0, best, s.queue, s.ctrl);
    LV_CK(cudaGetLastError());
    info->launches += 2;
    // Topo: persistent cooperative kernel over chain heads
    int occ = 0;
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
    A.tail = tail;
    A.len = len;
    A.hu = hu;
    A.indeg = s.indeg;
    A.best = best;
    A.queue = s.queue;
    A.ctrl = s.ctrl;
    A.narrow_max = kNarrowMax;
    A.wide_only = wide_only ? 1 : 0;
    void *args[] = {&A};
    LV_CK(cudaLaunchCooperativeKernel((const void *)k_kahn, grid, kKahnNT, args, 0, st));
    k_expand<<<gt, 256, 0, st>>>(n, J0, D0, best, level, s.ctrl);
    LV_CK(cudaGetLastError());
    info->launches += 2;
    int32_t ctrl[kCtrlInts];
    LV_CK(cudaMemcpyAsync(ctrl, s.ctrl, sizeof(ctrl), cudaMemcpyDeviceToHost, st));
    LV_CK(cudaStreamSynchronize(st));
    info->num_levels = ctrl[kMaxLevel] + 1;
    info->rounds = ctrl[kRound];
    info->wide_rounds = ctrl[kWide];
    info->narrow_rounds = ctrl[kNarrow];
    info->rank_rounds = contract ? ctrl[12] : 0;
    return cudaSuccess;
}

}  // namespace lusym
