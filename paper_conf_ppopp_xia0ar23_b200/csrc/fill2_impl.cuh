// fill2 traversal kernels (S3 count / S6 emit) for sm_100a — device code, instantiated per CTA
// size in fill2_nt*.cu.
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
// the dirty word range only).  Frontier levels are lists in shared memory, spilling to a
// per-CTA HBM region of capacity n.  Adjacency is read through an ELL-W copy of A without the
// diagonal (one 128/256-bit load per scanned vertex); vertices of larger degree are scanned by
// a whole warp from A's CSR.
#pragma once

#include "internal.h"

#include <climits>

namespace lusym {
namespace f2 {

#ifndef LUSYM_BATCH_TEST  // scan_level: load every neighbour's visited word before any atomic
#define LUSYM_BATCH_TEST 0    // (A/B on B200: 3.7% slower on cfg2, 5% on cfg5 — kept as a knob)
#endif
#ifndef LUSYM_FAST_SCAN  // scan_bits: warp-0 path for short ranges / full first windows
#define LUSYM_FAST_SCAN 1
#endif
#ifndef LUSYM_VPT  // frontier vertices per thread per round in plain BFS levels (1: scan_level)
#define LUSYM_VPT 1
#endif
#ifndef LUSYM_PRED_TAS  // test_and_mark as predicated straight-line code (shared bitmaps)
#define LUSYM_PRED_TAS 0
#endif
#ifndef LUSYM_ENC_ELL  // BFS of shared-map kernels reads neighbours pre-encoded as shared
#define LUSYM_ENC_ELL 1    // bitmap addresses (enc_slot), decoding only newly visited ones
#endif
#ifndef LUSYM_GB_DIRECT_ATOMIC  // HBM visited slots: test-and-set by the atomic alone
#define LUSYM_GB_DIRECT_ATOMIC 0
#endif
#ifndef LUSYM_GB_L1  // test_and_mark: HBM-slot pre-check loads cached in L1 (A/B knob)
#define LUSYM_GB_L1 0
#endif
#ifndef LUSYM_PREFETCH_NEXT  // prefetch a new frontier vertex's adjacency row into L1
#define LUSYM_PREFETCH_NEXT 0  // A/B: +7..15% slower (profiles/r02/ab_prefetch.log)
#endif
#ifndef LUSYM_WARP_EXIT  // warps past the end of a BFS level / threshold window leave early
#define LUSYM_WARP_EXIT 0  // A/B: +1.6..6.9% slower (profiles/r02/ab_wexit.log)
#endif
#ifndef LUSYM_ROUNDS  // scan_level (encoded neighbours): batch visited test, then atomics in
#define LUSYM_ROUNDS 0    // warp-uniform rounds of one candidate per lane (A/B: 12-17% slower)
#endif
#ifndef LUSYM_TAM  // test_and_mark with one shared bit mask (0: visited() then mark())
#define LUSYM_TAM 1
#endif
#ifndef LUSYM_THREADS_PER_SM_SMALL  // ... for CTAs of at most 128 threads
#define LUSYM_THREADS_PER_SM_SMALL LUSYM_THREADS_PER_SM
#endif
#ifndef LUSYM_THREADS_PER_SM  // register budget: 65536 / this
#define LUSYM_THREADS_PER_SM 2048
#endif

constexpr unsigned kFull = 0xffffffffu;
constexpr int kSmallWin = 32;  // threshold window after a window was cut short

struct Hdr {
    int row, minseed, diag, tns, newmin, ucnt, lmin, lmax;
    int cnt[3];
    int defer;
    long long stage_off;
    unsigned long long te, sv, spills;  // statistics of this CTA (thread 0 / shared atomics)
    int scan[40];
    // asynchronous BFS (bfs_async): pool lock, pool entries, vertices discovered and not yet
    // expanded (in a ring, in the pool or being expanded), idle warps
    int alock, ptop, outst, idle;
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

// Visited bitmap of the row in flight.
//   kVisSmem   : every word in shared memory
//   kVisSplit  : words [0, lbw) in shared memory, the rest in the CTA's HBM slot — row classes
//                (Alg. 4): rows below lbw*32 keep their whole BFS region
//                (all vertices < src) in shared memory, only pattern marks above it go to HBM
//   kVisGlobal : every word in the CTA's HBM slot
// Shared words are XOR-swizzled inside each group of 32, so words 32 (or a multiple of 32)
// apart — grid neighbours at +-k for k a multiple of 1024 — fall into different banks.
template <int VIS>
struct VisMap {
    uint32_t *s;  // shared part
    uint32_t *g;  // HBM slot (word index = vertex >> 5)
    int lbw;      // words held in shared memory (kVisSplit)
    int nw;       // shared visited words (the level-1 summary follows them)
    uint32_t ssum;  // shared address of the level-1 summary (from the runtime window base)
};


template <int VIS>
__device__ __forceinline__ int phys(const VisMap<VIS> &m, int w)
{
    if (!LUSYM_SWZ) return w;
    return w ^ ((w >> 5) & 31);
}

template <int VIS>
__device__ __forceinline__ bool in_smem(const VisMap<VIS> &m, int w)
{
    if (VIS == kVisGlobal) return false;
    if (VIS == kVisSmem) return true;
    return w < m.lbw;
}

// The shared visited words sit at a constant offset of the CTA's shared window: dynamic shared
// memory starts right after the 1 KB system reservation (checked at kernel start, see
// check_smem_base), then the header.  Addressing them as [4*word + immediate] keeps the window
// base out of the registers of the slot loop (at 32 registers/thread the compiler would
// otherwise rematerialise it for every neighbour).
constexpr uint32_t kDynSmemBase = 0x400;
constexpr uint32_t kBmShared = kDynSmemBase + kHdrBytes;

__device__ __forceinline__ uint32_t lds_bm(int pw)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(pw * 4), "n"(kBmShared) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t atom_or_bm(int pw, uint32_t b)
{
    uint32_t old;
    asm volatile("atom.shared.or.b32 %0, [%1+%2], %3;"
                 : "=r"(old)
                 : "r"(pw * 4), "n"(kBmShared), "r"(b)
                 : "memory");
    return old;
}

// The host probes the window base once per device (fill2_smem_base_ok) and plans only
// kVisGlobal classes when it is not kDynSmemBase, so this trap is a last-resort assertion.
__device__ __forceinline__ void check_smem_base(const unsigned char *smem)
{
    if (threadIdx.x == 0 && (uint32_t)__cvta_generic_to_shared(smem) != kDynSmemBase) __trap();
}

// shared byte address of the level-1 summary (taken from the actual window, so kVisGlobal
// kernels do not depend on where the dynamic shared memory starts)
template <int VIS>
__device__ __forceinline__ uint32_t summary_saddr(const VisMap<VIS> &m)
{
    return m.ssum;
}

template <int VIS>
__device__ __forceinline__ uint32_t bm_word(const VisMap<VIS> &m, int w)
{
    if (in_smem(m, w)) return lds_bm(phys<VIS>(m, w));
    return __ldcg(m.g + w);
}

template <int VIS>
__device__ __forceinline__ void bm_zero(const VisMap<VIS> &m, int w)
{
    if (in_smem(m, w))
        m.s[phys<VIS>(m, w)] = 0;
    else
        m.g[w] = 0;
}

template <int VIS>
__device__ __forceinline__ bool visited(const VisMap<VIS> &m, int v)
{
    return (bm_word(m, v >> 5) >> (v & 31)) & 1u;
}

// test-and-set (reading R26): true iff this call set the bit.  The level-1 summary sm gets bit
// w when visited word w first becomes non-zero, so scans and clears skip empty stretches.
template <int VIS>
__device__ __forceinline__ bool mark(const VisMap<VIS> &m, uint32_t *sm, int v)
{
    const uint32_t b = 1u << (v & 31);
    const int w = v >> 5;
    const uint32_t old = in_smem(m, w) ? atom_or_bm(phys<VIS>(m, w), b) : atomicOr(m.g + w, b);
    if (old == 0)
        asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(summary_saddr(m) + (uint32_t)(v >> 10) * 4u),
                     "r"(1u << (w & 31))
                     : "memory");
    (void)sm;
    return !(old & b);
}

// visited test, then test-and-set only if the bit looked clear (the atomic decides); the bit
// mask is computed once for both.  True iff this call set the bit.
template <int VIS>
__device__ __forceinline__ bool test_and_mark(const VisMap<VIS> &m, uint32_t *sm, int v)
{
#if LUSYM_PRED_TAS
    if constexpr (VIS == kVisSmem) {
        // straight-line: a plain shared load (the compiler may batch the W loads of a vertex),
        // then the atomic and the summary update as predicated instructions — no branch and
        // no reconvergence barrier per neighbour
        const uint32_t b = 1u << (v & 31);
        const int w = v >> 5;
        const uint32_t a = (uint32_t)phys<VIS>(m, w) * 4u;
        uint32_t word;
        asm("ld.shared.u32 %0, [%1+%2];" : "=r"(word) : "r"(a), "n"(kBmShared));
        uint32_t old;
        asm volatile(
            "{\n\t.reg .pred p, q;\n\t"
            "setp.eq.u32 p, %2, 0;\n\t"
            "mov.u32 %0, %3;\n\t"
            "@p atom.shared.or.b32 %0, [%1+%4], %3;\n\t"
            "setp.eq.and.u32 q, %0, 0, p;\n\t"
            "@q red.shared.or.b32 [%5], %6;\n\t}"
            : "=&r"(old)
            : "r"(a), "r"(word & b), "r"(b), "n"(kBmShared),
              "r"(summary_saddr(m) + (uint32_t)(v >> 10) * 4u), "r"(1u << (w & 31))
            : "memory");
        return !(old & b);  // visited: old = b
    }
#endif
#if LUSYM_TAM
    const uint32_t b = 1u << (v & 31);
    const int w = v >> 5;
    const bool sh = in_smem(m, w);
#if LUSYM_GB_DIRECT_ATOMIC
    if (VIS == kVisGlobal) {
        // HBM slot: one L2 round trip (the atomic returns the old word) instead of a load
        // followed, for an unvisited bit, by the atomic
        const uint32_t old = atomicOr(m.g + w, b);
        if (old == 0)
            asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(summary_saddr(m) + (uint32_t)(v >> 10) * 4u),
                         "r"(1u << (w & 31))
                         : "memory");
        return !(old & b);
    }
#endif
    // (LUSYM_GB_L1: the HBM slot's pre-check through L1.  Only this CTA writes its slot and
    // bits only get set during a row, so a stale L1 copy can only miss bits, which the atomic
    // then decides; the per-row clears are this CTA's own stores.)
    const uint32_t word = sh ? lds_bm(phys<VIS>(m, w))
                             : (LUSYM_GB_L1 ? __ldca(m.g + w) : __ldcg(m.g + w));
    if (word & b) return false;
    const uint32_t old = sh ? atom_or_bm(phys<VIS>(m, w), b) : atomicOr(m.g + w, b);
    if (old == 0)
        asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(summary_saddr(m) + (uint32_t)(v >> 10) * 4u),
                     "r"(1u << (w & 31))
                     : "memory");
    (void)sm;
    return !(old & b);
#else
    return !visited(m, v) && mark(m, sm, v);
#endif
}

// Encoded neighbour of the shared-map kernels (built by k_build_ell_enc): e = phys(v >> 5) << 7
// | (v & 31).  e >> 5 is the byte offset of v's visited word (phys << 2 exactly: the bit index
// shifts out), and a funnel shift by e uses only its low 5 bits, the bit of v — so the common
// visited test is one shift, one shared load and one bit test; only a newly visited neighbour
// is decoded back to v (the swizzle is an involution on the word index).
__device__ __forceinline__ int dec_slot(int e)
{
    int pw = e >> 7;
    if (LUSYM_SWZ) pw ^= (pw >> 5) & 31;
    return (pw << 5) | (e & 31);
}

// test-and-set of the encoded neighbour e (kVisSmem): true iff this call set the bit; *v = the
// decoded vertex when true
template <int VIS>
__device__ __forceinline__ bool test_and_mark_enc(const VisMap<VIS> &m, int e, int *v)
{
    const uint32_t off = (uint32_t)e >> 5;
    uint32_t word;
    asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(word) : "r"(off), "n"(kBmShared) : "memory");
    const uint32_t b = 1u << (e & 31);
    if (word & b) return false;
    uint32_t old;
    asm volatile("atom.shared.or.b32 %0, [%1+%2], %3;"
                 : "=r"(old) : "r"(off), "n"(kBmShared), "r"(b) : "memory");
    if (old & b) return false;
    const int x = dec_slot(e);
    *v = x;
    if (old == 0)
        asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(summary_saddr(m) + (uint32_t)(x >> 10) * 4u),
                     "r"(1u << ((x >> 5) & 31))
                     : "memory");
    return true;
}

// the set half of test_and_mark_enc (the bit looked clear): true iff this call set it
template <int VIS>
__device__ __forceinline__ bool set_enc(const VisMap<VIS> &m, int e, int *v)
{
    const uint32_t off = (uint32_t)e >> 5;
    const uint32_t b = 1u << (e & 31);
    uint32_t old;
    asm volatile("atom.shared.or.b32 %0, [%1+%2], %3;"
                 : "=r"(old) : "r"(off), "n"(kBmShared), "r"(b) : "memory");
    if (old & b) return false;
    const int x = dec_slot(e);
    *v = x;
    if (old == 0)
        asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(summary_saddr(m) + (uint32_t)(x >> 10) * 4u),
                     "r"(1u << ((x >> 5) & 31))
                     : "memory");
    return true;
}

// ELL slots W in {4, 6, 8}; rows are stored 4 (W = 4) or 8 (W = 6, 8) entries wide.  A light
// row of degree < W is padded with the vertex itself, which is always visited when its row is
// read, so the slot loop needs no sentinel test.
template <int W>
__host__ __device__ constexpr int ell_stride()
{
    return W <= 4 ? 4 : 8;
}

template <int W>
__device__ __forceinline__ void load_nb(const int32_t *ell, int f, int (&nb)[ell_stride<W>()])
{
    if constexpr (ell_stride<W>() == 8) {
        // one 256-bit load per adjacency row (LDG.E.256 on sm_100a)
        asm("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
            : "=r"(nb[0]), "=r"(nb[1]), "=r"(nb[2]), "=r"(nb[3]), "=r"(nb[4]), "=r"(nb[5]),
              "=r"(nb[6]), "=r"(nb[7])
            : "l"(ell + (size_t)f * 8));
    } else {
        const int4 a = __ldg(reinterpret_cast<const int4 *>(ell + (size_t)f * 4));
        nb[0] = a.x; nb[1] = a.y; nb[2] = a.z; nb[3] = a.w;
    }
}

// Traversed edges of a scanned light vertex (reading R24: its full row, diagonal included):
// the slots that are not its own padding, + 1 for the diagonal (build_ell makes every row
// without a diagonal a heavy record, whose CSR length is counted instead).  pad = the padding
// value of the row: the vertex itself, encoded as the slots are.
template <int W>
__device__ __forceinline__ int row_edges(const int (&nb)[ell_stride<W>()], int pad)
{
    int d = 1;
#pragma unroll
    for (int s = 0; s < W; ++s) d += nb[s] != pad;
    return d;
}

__device__ __forceinline__ int enc_vertex(int v)
{
    int pw = v >> 5;
    if (LUSYM_SWZ) pw ^= (pw >> 5) & 31;
    return (pw << 7) | (v & 31);
}

// store a frontier entry (shared memory, HBM past q)
__device__ __forceinline__ void put(int pos, int w, int32_t *NF, int32_t *gNF, int q)
{
    if (pos < q)
        NF[pos] = w;
    else
        gNF[pos] = w;
}

__device__ __forceinline__ int64_t heavy_off(int lo, int hi)
{
    return (int64_t)(uint32_t)lo | ((int64_t)hi << 32);
}

// warp-aggregated append to a list (smem, spilling to HBM past q entries)
__device__ __forceinline__ void push(bool pred, int w, int *cnt, int32_t *NF, int32_t *gNF, int q)
{
    const unsigned b = __ballot_sync(kFull, pred);
    if (b == 0) return;
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(b) - 1;
    int base = 0;
    if (lane == leader) base = atomicAdd(cnt, __popc(b));
    base = __shfl_sync(kFull, base, leader);
    if (pred) put(base + __popc(b & ((1u << lane) - 1u)), w, NF, gNF, q);
}

// Smallest visited word index >= w0 whose summary bit is set (may exceed whi within the last
// summary word), INT_MAX if none up to whi.  Block-uniform; sred: NT/32 ints of scratch.
template <int NT>
__device__ int next_word(const uint32_t *sm, int w0, int whi, int *sred)
{
    const int shi = whi >> 5;
    for (int sb = w0 >> 5; sb <= shi; sb += NT) {
        const int sidx = sb + (int)threadIdx.x;
        int cand = INT_MAX;
        if (sidx <= shi) {
            uint32_t sw = sm[sidx];
            if (sidx == (w0 >> 5)) sw &= kFull << (w0 & 31);
            if (sw) cand = (sidx << 5) + __ffs(sw) - 1;
        }
        cand = __reduce_min_sync(kFull, cand);
        if ((threadIdx.x & 31) == 0) sred[threadIdx.x >> 5] = cand;
        __syncthreads();
        int r = INT_MAX;
#pragma unroll
        for (int k = 0; k < NT / 32; ++k) r = min(r, sred[k]);
        __syncthreads();
        if (r != INT_MAX) return r;
    }
    return INT_MAX;
}

// Set bits of (bm & ~dm) in [lo, hi) (dm may be null), in increasing order.  Returns how many
// there are (at most cap when CAPPED).  WRITE: stores them at dst[base + k] for base + k < dcap.
// One visited word per thread per chunk; on ranges wider than a chunk the level-1 summary sm
// skips empty stretches before each chunk.  Block-uniform.
template <int NT, int VIS, bool WRITE, bool CAPPED>
__device__ int scan_bits(const VisMap<VIS> &bm, const uint32_t *sm, const uint32_t *dm, int lo,
                         int hi, int32_t *dst, int64_t base, int64_t dcap, int cap, int *sscan)
{
    if (lo >= hi) return 0;
    const int wlo = lo >> 5, whi = (hi - 1) >> 5;
#if LUSYM_FAST_SCAN
    // warp 0 alone, two barriers instead of a block scan: the range fits 32 words, or (collect)
    // its first 32 words already hold cap set bits — the common case on the serial threshold
    // chain of heavy rows, where the pointer advances by a few words per window
    if (whi - wlo < 32 || CAPPED) {
        if (threadIdx.x < 32) {
            const int lane = threadIdx.x;
            const int w = wlo + lane;
            uint32_t word = 0;
            if (w <= whi) {
                word = bm_word(bm, w);
                if (w == wlo) word &= kFull << (lo & 31);
                if (w == whi) {
                    const int hb = (hi - 1) & 31;
                    word &= (hb == 31) ? kFull : ((2u << hb) - 1u);
                }
                if (dm && word) word &= ~__ldcg(dm + w);
            }
            const int c = __popc(word);
            int inc = c;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int y = __shfl_up_sync(kFull, inc, o);
                if (lane >= o) inc += y;
            }
            const int total = __shfl_sync(kFull, inc, 31);
            const bool ok = whi - wlo < 32 || total >= cap;
            if (ok && WRITE) {
                int pos = inc - c;
                for (; word && !(CAPPED && pos >= cap); word &= word - 1, ++pos) {
                    const int64_t o = base + pos;
                    if (o < dcap) dst[o] = (w << 5) + __ffs(word) - 1;
                }
            }
            if (lane == 0) sscan[33] = ok ? total : -1;
        }
        __syncthreads();
        const int r = sscan[33];
        __syncthreads();
        if (r >= 0) return CAPPED && r > cap ? cap : r;
    }
#endif
    const bool wide = whi - wlo >= NT;
    int count = 0;
    for (int w0 = wlo; w0 <= whi; w0 += NT) {
        if (wide) {
            w0 = next_word<NT>(sm, w0, whi, sscan);
            if (w0 > whi) break;
        }
        const int w = w0 + (int)threadIdx.x;
        uint32_t word = 0;
        if (w <= whi) {
            word = bm_word(bm, w);
            if (w == wlo) word &= kFull << (lo & 31);
            if (w == whi) {
                const int hb = (hi - 1) & 31;
                word &= (hb == 31) ? kFull : ((2u << hb) - 1u);
            }
            if (dm && word) word &= ~__ldcg(dm + w);
        }
        int total;
        int pos = count + block_scan_excl<NT>(__popc(word), sscan, total);
        if (WRITE)
            for (; word; word &= word - 1, ++pos) {
                const int64_t o = base + pos;
                if (o < dcap) dst[o] = (w << 5) + __ffs(word) - 1;
            }
        count += total;
        if (CAPPED && count >= cap) break;
    }
    if (WRITE) __syncthreads();
    return CAPPED && count > cap ? cap : count;
}

// Pending thresholds not yet finished: the first cap set bits of bm & ~dm in [lo, hi), sorted.
template <int NT, int VIS>
__device__ __forceinline__ int collect(const VisMap<VIS> &bm, const uint32_t *sm, const uint32_t *dm,
                                       int lo, int hi, int32_t *out, int cap, int *sscan)
{
    return scan_bits<NT, VIS, true, true>(bm, sm, dm, lo, hi, out, 0, cap, cap, sscan);
}

// Count the set bits in [lo, hi) and, if WRITE, store them in increasing order at dst[base ..]
// (bounded by cap).  Returns the count.
template <int NT, int VIS, bool WRITE>
__device__ __forceinline__ int emit_range(const VisMap<VIS> &bm, const uint32_t *sm, int lo, int hi,
                                          int32_t *dst, int base, int64_t cap, int *sscan)
{
    return scan_bits<NT, VIS, WRITE, false>(bm, sm, nullptr, lo, hi, dst, base, cap, 0, sscan);
}

// Zero the visited words [wlo, whi] and their summary bits (walk the summary if wide).
template <int NT, int VIS>
__device__ void clear_words(const VisMap<VIS> &bm, uint32_t *sm, int wlo, int whi)
{
    if (whi < wlo) return;
    if (whi - wlo < 4 * NT) {
        for (int w = wlo + (int)threadIdx.x; w <= whi; w += NT) bm_zero(bm, w);
    } else {
        for (int sidx = (wlo >> 5) + (int)threadIdx.x; sidx <= (whi >> 5); sidx += NT)
            for (uint32_t t = sm[sidx]; t; t &= t - 1) bm_zero(bm, (sidx << 5) + __ffs(t) - 1);
    }
    __syncthreads();
    for (int sidx = (wlo >> 5) + (int)threadIdx.x; sidx <= (whi >> 5); sidx += NT) sm[sidx] = 0;
}

struct RowAcc {
    int ucnt, lmin, lmax;
};

// Scan the vertices L[0..cnt) (smem, HBM past q) of one BFS level below t0: test-and-set every
// neighbour; new ones below t0 form the next level (appended to NF), new ones above t0 are
// pattern entries (L130-147).  Self-continuation (reading R5, the order below a threshold is
// free): a lane that discovered new vertices expands the first of them itself in the next
// round, up to p.kloc rounds, so a BFS front advances more than one step per level barrier;
// only the other discoveries go through the next-level queue.  Worth it only where a row has
// an SM to itself and waits on each level's latency (the planner sets kloc per row class):
// with many rows per SM the extra rounds, in which lanes drop out, cost issue slots.
template <int NT, int W, int VIS, bool SC, int MODE>
__device__ __forceinline__ void scan_level(const Fill2Params &p, Hdr &h, const VisMap<VIS> &bm,
                                           uint32_t *sm, const int32_t *L, const int32_t *gL,
                                           int cnt, int *ncnt, int32_t *NF, int32_t *gNF,
                                           const int i, const int t0, RowAcc &a)
{
    const int tid = threadIdx.x, lane = tid & 31;
    const unsigned lt = (1u << lane) - 1u;
    const uint32_t ncnt_s = (uint32_t)__cvta_generic_to_shared(ncnt);
    unsigned nloc = 0;  // vertices expanded by self-continuation (statistics, lane 0)
    unsigned long long te_loc = 0;  // traversed edges of light vertices (p.count_te)
    for (int base = 0; base < cnt; base += NT) {
#if LUSYM_WARP_EXIT
        // a warp past the end of the level leaves (warp-uniform) instead of running the body
        // with no valid lane: levels narrower than the CTA are most of a BFS's levels
        if (base + (tid & ~31) >= cnt) break;
#endif
        const int k = base + tid;
        bool valid = k < cnt;
        int f = valid ? (k < p.q ? L[k] : __ldcg(gL + k)) : 0;
      for (int r = 0;; ++r) {
        int nb[ell_stride<W>()];
#if !LUSYM_NO_NB_INIT
#pragma unroll
        for (int s = 0; s < ell_stride<W>(); ++s) nb[s] = 0;
#endif
        bool heavy = false;
        // new frontier vertices of this thread: the first three stay in registers (f0..f2) for
        // one warp-aggregated append (a grid vertex has up to three neighbours further from
        // the BFS source); further ones (rare) are appended one by one
        int c = 0, f0 = 0, f1 = 0, f2 = 0;
        const bool enc = LUSYM_ENC_ELL && VIS == kVisSmem && p.elle != nullptr;
        uint32_t um = 0;  // LUSYM_ROUNDS: slots whose neighbour looked unvisited
        if (valid) {
            load_nb<W>(enc ? p.elle : p.ell, f, nb);
            heavy = nb[0] == kHeavy;
            if constexpr (MODE == kCount)  // the statistics pass only (LU_F_COUNT_TE)
                if (p.count_te && !heavy) te_loc += row_edges<W>(nb, enc ? enc_vertex(f) : f);
            if (enc && !heavy && LUSYM_ROUNDS) {
                // every slot's visited bit first (straight-line, no branch per slot); the
                // candidates are test-and-set after this block in warp-uniform rounds
#pragma unroll
                for (int s = 0; s < W; ++s) {
                    uint32_t word;
                    asm volatile("ld.shared.u32 %0, [%1+%2];"
                                 : "=r"(word) : "r"((uint32_t)nb[s] >> 5), "n"(kBmShared)
                                 : "memory");
                    um |= (((word >> (nb[s] & 31)) & 1u) ^ 1u) << s;
                }
            } else if (enc && !heavy) {
#pragma unroll
                for (int s = 0; s < W; ++s) {
                    int w;
                    if (test_and_mark_enc(bm, nb[s], &w)) {
                        if (w < t0) {
#if LUSYM_PREFETCH_NEXT
                            // the next level reads w's adjacency: start it towards L1 now
                            asm volatile("prefetch.global.L1 [%0];" ::"l"(
                                p.elle + (size_t)w * ell_stride<W>()));
#endif
                            if (c == 3) {
                                put(atomicAdd(ncnt, 1), w, NF, gNF, p.q);
                            } else {
                                f2 = f1;
                                f1 = f0;
                                f0 = w;
                                ++c;
                            }
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
            } else if (!heavy) {
                // all W visited words first (independent loads in flight together), then the
                // test-and-set only on the slots that looked unvisited (the atomic decides)
                uint32_t um = 0;
#pragma unroll
                for (int s = 0; s < W; ++s) {
#if LUSYM_BATCH_TEST
                    const uint32_t wd = bm_word(bm, nb[s] >> 5);
                    um |= ((~wd >> (nb[s] & 31)) & 1u) << s;
#else
                    um |= 1u << s;
#endif
                }
#pragma unroll
                for (int s = 0; s < W; ++s) {
                    const int w = nb[s];
                    if ((um >> s & 1u) &&
                        (LUSYM_BATCH_TEST ? mark(bm, sm, w) : test_and_mark(bm, sm, w))) {
                        if (w < t0) {
                            if (c == 3) {
                                put(atomicAdd(ncnt, 1), w, NF, gNF, p.q);
                            } else {
                                f2 = f1;
                                f1 = f0;
                                f0 = w;
                                ++c;
                            }
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
            }
        }
        if (LUSYM_ROUNDS && enc) {
            // the candidates, one per lane per round: the atomic path is issued once per round
            // for the warp instead of once per slot
            while (__any_sync(kFull, um != 0)) {
                if (um) {
                    const int s0 = __ffs(um) - 1;
                    um &= um - 1;
                    int e = nb[0];
#pragma unroll
                    for (int s = 1; s < W; ++s)
                        if (s == s0) e = nb[s];
                    int w;
                    if (set_enc(bm, e, &w)) {
                        if (w < t0) {
                            if (c == 3) {
                                put(atomicAdd(ncnt, 1), w, NF, gNF, p.q);
                            } else {
                                f2 = f1;
                                f1 = f0;
                                f0 = w;
                                ++c;
                            }
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
            }
        }
        // SC: keep f0 for the next round, append the rest
        bool keep = false;
        if constexpr (SC) {
            keep = r < p.kloc && c > 0;
            if (keep) {
                --c;
                const int t = f0;
                f0 = f1;
                f1 = f2;
                f2 = t;
            }
        }
        const unsigned b1 = __ballot_sync(kFull, c & 1), b2 = __ballot_sync(kFull, c & 2);
        if (b1 | b2) {
            const int tot = __popc(b1) + 2 * __popc(b2);
            int wbase = 0;
            // one shared atomic by lane 0 (inline PTX: no compiler re-aggregation around it)
            if (lane == 0)
                asm volatile("atom.shared.add.u32 %0, [%1], %2;"
                             : "=r"(wbase) : "r"(ncnt_s), "r"(tot) : "memory");
            wbase = __shfl_sync(kFull, wbase, 0);
            const int pos = wbase + __popc(b1 & lt) + 2 * __popc(b2 & lt);
            if (wbase + tot <= p.q) {  // warp-uniform: the whole append lands in shared memory
                if (c) NF[pos] = f0;
                if (c >= 2) NF[pos + 1] = f1;
                if (c == 3) NF[pos + 2] = f2;
            } else {
                if (c) put(pos, f0, NF, gNF, p.q);
                if (c >= 2) put(pos + 1, f1, NF, gNF, p.q);
                if (c == 3) put(pos + 2, f2, NF, gNF, p.q);
            }
        }
        // heavy vertices (degree > W): one warp each, over A's CSR row
        unsigned hm = __ballot_sync(kFull, valid && heavy);
        while (hm) {
            const int src = __ffs(hm) - 1;
            hm &= hm - 1;
            const int len = __shfl_sync(kFull, nb[1], src);
            const int64_t off =
                heavy_off(__shfl_sync(kFull, nb[2], src), __shfl_sync(kFull, nb[3], src));
            if (lane == 0) atomicAdd(&h.te, (unsigned long long)len);
            for (int eb = 0; eb < len; eb += 32) {
                const int e = eb + lane;
                bool fr = false;
                int w = -1;
                if (e < len) {
                    w = __ldg(p.ci + off + e);
                    if (test_and_mark(bm, sm, w)) {
                        if (w < t0) {
                            fr = true;
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
                push(fr, w, ncnt, NF, gNF, p.q);
            }
        }
        if constexpr (!SC) {
            break;
        } else {
            const unsigned kb = __ballot_sync(kFull, keep);
            if (!kb) break;
            nloc += __popc(kb);
            valid = keep;
            f = f2;
        }
      }
    }
    if (SC && lane == 0 && nloc) atomicAdd(&h.sv, (unsigned long long)nloc);
    if (MODE == kCount && p.count_te) {
#pragma unroll
        for (int o = 16; o; o >>= 1) te_loc += __shfl_xor_sync(kFull, te_loc, o);
        if (lane == 0 && te_loc) atomicAdd(&h.te, te_loc);
    }
}

// Plain level-synchronous variant of scan_level with VPT frontier vertices per thread per
// round (LUSYM_VPT > 1): the per-round overhead (queue index, ballots, shared append) is
// shared by VPT vertices; new frontier vertices still collect in f0..f2 across them.
template <int NT, int W, int VIS, int VPT>
__device__ __forceinline__ void scan_level_multi(const Fill2Params &p, Hdr &h,
                                                 const VisMap<VIS> &bm, uint32_t *sm,
                                                 const int32_t *L, const int32_t *gL, int cnt,
                                                 int *ncnt, int32_t *NF, int32_t *gNF,
                                                 const int i, const int t0, RowAcc &a)
{
    const int tid = threadIdx.x, lane = tid & 31;
    const unsigned lt = (1u << lane) - 1u;
    const uint32_t ncnt_s = (uint32_t)__cvta_generic_to_shared(ncnt);
    for (int base = 0; base < cnt; base += NT * VPT) {
        int c = 0, f0 = 0, f1 = 0, f2 = 0;
#pragma unroll
        for (int v = 0; v < VPT; ++v) {
            const int k = base + v * NT + tid;
            const bool valid = k < cnt;
            int nb[ell_stride<W>()];
#pragma unroll
            for (int s = 0; s < ell_stride<W>(); ++s) nb[s] = 0;
            bool heavy = false;
            if (valid) {
                const int f = k < p.q ? L[k] : __ldcg(gL + k);
                load_nb<W>(p.ell, f, nb);
                heavy = nb[0] == kHeavy;
                if (!heavy) {
#pragma unroll
                    for (int s = 0; s < W; ++s) {
                        const int w = nb[s];
                        if (test_and_mark(bm, sm, w)) {
                            if (w < t0) {
                                if (c == 3) {
                                    put(atomicAdd(ncnt, 1), w, NF, gNF, p.q);
                                } else {
                                    f2 = f1;
                                    f1 = f0;
                                    f0 = w;
                                    ++c;
                                }
                            } else if (w > i) {
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
                const int len = __shfl_sync(kFull, nb[1], src);
                const int64_t off =
                    heavy_off(__shfl_sync(kFull, nb[2], src), __shfl_sync(kFull, nb[3], src));
                if (lane == 0) atomicAdd(&h.te, (unsigned long long)len);
                for (int eb = 0; eb < len; eb += 32) {
                    const int e = eb + lane;
                    bool fr = false;
                    int w = -1;
                    if (e < len) {
                        w = __ldg(p.ci + off + e);
                        if (test_and_mark(bm, sm, w)) {
                            if (w < t0) {
                                fr = true;
                            } else if (w > i) {
                                ++a.ucnt;
                                a.lmax = max(a.lmax, w);
                            }
                        }
                    }
                    push(fr, w, ncnt, NF, gNF, p.q);
                }
            }
        }
        const unsigned b1 = __ballot_sync(kFull, c & 1), b2 = __ballot_sync(kFull, c & 2);
        if (b1 | b2) {
            const int tot = __popc(b1) + 2 * __popc(b2);
            int wbase = 0;
            if (lane == 0)
                asm volatile("atom.shared.add.u32 %0, [%1], %2;"
                             : "=r"(wbase) : "r"(ncnt_s), "r"(tot) : "memory");
            wbase = __shfl_sync(kFull, wbase, 0);
            const int pos = wbase + __popc(b1 & lt) + 2 * __popc(b2 & lt);
            if (wbase + tot <= p.q) {
                if (c) NF[pos] = f0;
                if (c >= 2) NF[pos + 1] = f1;
                if (c == 3) NF[pos + 2] = f2;
            } else {
                if (c) put(pos, f0, NF, gNF, p.q);
                if (c >= 2) put(pos + 1, f1, NF, gNF, p.q);
                if (c == 3) put(pos + 2, f2, NF, gNF, p.q);
            }
        }
    }
}

// ---- Asynchronous below-threshold traversal (reading R5: which vertices below t0 are reached
// is fixed, the order is free, so no level barrier is needed).  Each warp expands up to 32
// vertices at a time from its own ring in shared memory (head/tail in registers: no atomics on
// the queue) and appends what they discover to the same ring.  A warp whose ring is empty takes
// work from the CTA's pool (a stack in the rest of the queues' shared memory, continued in the
// HBM frontier spill region, under a shared-memory lock); a warp with a long ring donates half of it while other warps are idle, and a warp
// whose ring would overflow moves its ring to the pool.  h.outst counts the vertices
// discovered and not yet expanded (rings + pool + being expanded); the traversal is over when
// it is 0.  A warp's children are added to h.outst before any of them can reach another warp
// (at the latest when the warp donates), so it never reads 0 while work is left.

// lane 0 takes the pool lock; every lane returns after it is held
__device__ __forceinline__ void pool_lock(Hdr &h)
{
    if ((threadIdx.x & 31) == 0) {
        while (atomicCAS(&h.alock, 0, 1) != 0) __nanosleep(32);
        __threadfence_block();
    }
    __syncwarp();
}

// every lane's pool and ring accesses are ordered before lane 0 releases the lock
__device__ __forceinline__ void pool_unlock(Hdr &h)
{
    __threadfence_block();
    __syncwarp();
    if ((threadIdx.x & 31) == 0) atomicExch(&h.alock, 0);
    __syncwarp();
}

// Move the cnt oldest entries of the warp's ring to the pool (warp-uniform).  pend = children
// appended since the warp last updated h.outst: they are counted before the pool publishes them.
__device__ __forceinline__ void ring_donate(Hdr &h, int32_t *ring, int R, int &head, int cnt,
                                            int32_t *spool, int pcap, int32_t *pool, int &pend,
                                            unsigned long long &nspill)
{
    __syncwarp();
    pool_lock(h);
    const int lane = threadIdx.x & 31;
    int top = 0;
    if (lane == 0) {
        if (pend) atomicAdd(&h.outst, pend);
        top = *(volatile int *)&h.ptop;
    }
    top = __shfl_sync(kFull, top, 0);
    for (int k = lane; k < cnt; k += 32) {
        const int x = top + k, v = ring[(head + k) & (R - 1)];
        if (x < pcap)
            spool[x] = v;
        else
            __stcg(pool + (x - pcap), v);
    }
    __threadfence_block();
    if (lane == 0) *(volatile int *)&h.ptop = top + cnt;
    pool_unlock(h);
    pend = 0;
    head += cnt;
    if (top + cnt > pcap) nspill += (unsigned long long)(top + cnt - max(top, pcap));
}

// warp-aggregated append of v (lanes with pred; b = their ballot) to the warp's ring
__device__ __forceinline__ void ring_append(Hdr &h, bool pred, unsigned b, int v, int32_t *ring,
                                            int R, int &head, int &tail, int32_t *spool, int pcap,
                                            int32_t *pool, int &pend, unsigned long long &nspill)
{
    const int tot = __popc(b);
    if (tail - head + tot > R)
        ring_donate(h, ring, R, head, tail - head, spool, pcap, pool, pend, nspill);
    if (pred) ring[(tail + __popc(b & ((1u << (threadIdx.x & 31)) - 1u))) & (R - 1)] = v;
    tail += tot;
    pend += tot;
}

template <int NT, int W, int VIS, int MODE>
__device__ void bfs_async(const Fill2Params &p, Hdr &h, const VisMap<VIS> &bm, uint32_t *sm,
                          int32_t *qA, const int i, const int t0, RowAcc &a)
{
    constexpr int NW = NT / 32;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int R = p.aring;  // ring entries per warp (a power of two >= 64)
    int32_t *ring = qA + wid * R;
    // the pool: the rest of the two frontier queues' shared memory, then the HBM spill region
    int32_t *spool = qA + NW * R;
    const int pcap = 2 * p.q - NW * R;
    int32_t *pool = p.gspill + (size_t)blockIdx.x * 2 * p.spill_cap;
    if (threadIdx.x == 0) {
        h.alock = 0;
        h.ptop = 0;
        h.outst = 1;
        h.idle = NW - 1;
        ring[0] = t0;
    }
    __syncthreads();
    int head = 0, tail = wid == 0 ? 1 : 0;  // warp-uniform ring positions
    int pend = 0;                           // children not yet added to h.outst (uniform)
    unsigned long long nproc = 0, nspill = 0, te_loc = 0;
    bool idle = wid != 0;
    const bool enc = LUSYM_ENC_ELL && VIS == kVisSmem && p.elle != nullptr;
    for (;;) {
        if (tail == head) {
            // no work of its own: take from the pool, or stop when nothing is left anywhere
            if (!idle) {
                idle = true;
                if (lane == 0) atomicAdd(&h.idle, 1);
            }
            int got = 0;
            for (;;) {
                int top = 0, out = 0;
                if (lane == 0) {
                    top = *(volatile int *)&h.ptop;
                    out = *(volatile int *)&h.outst;
                }
                top = __shfl_sync(kFull, top, 0);
                out = __shfl_sync(kFull, out, 0);
                if (top > 0) {
                    pool_lock(h);
                    int t = 0;
                    if (lane == 0) {
                        t = *(volatile int *)&h.ptop;
                        got = min(t, 32);
                        *(volatile int *)&h.ptop = t - got;
                    }
                    t = __shfl_sync(kFull, t, 0);
                    got = __shfl_sync(kFull, got, 0);
                    if (lane < got) {
                        const int x = t - got + lane;
                        ring[(tail + lane) & (R - 1)] =
                            x < pcap ? spool[x] : __ldcg(pool + (x - pcap));
                    }
                    pool_unlock(h);
                    if (got) break;
                } else if (out == 0) {
                    break;
                }
                __nanosleep(p.asleep);
            }
            if (!got) break;
            tail += got;
            idle = false;
            if (lane == 0) atomicSub(&h.idle, 1);
        } else if (tail - head > p.akeep + 8) {
            // other warps idle and the pool nearly empty: keep akeep entries, hand over the rest
            int ask = 0;
            if (lane == 0)
                ask = *(volatile int *)&h.idle > 0 && *(volatile int *)&h.ptop < 32;
            if (__shfl_sync(kFull, ask, 0))
                ring_donate(h, ring, R, head, tail - head - p.akeep, spool, pcap, pool, pend,
                            nspill);
        }
        __syncwarp();
        const int m = min(tail - head, 32);
        const bool valid = lane < m;
        const int f = valid ? ring[(head + lane) & (R - 1)] : 0;
        head += m;
        nproc += (unsigned long long)m;
        int nb[ell_stride<W>()];
#pragma unroll
        for (int s = 0; s < ell_stride<W>(); ++s) nb[s] = 0;
        bool heavy = false;
        unsigned newm = 0;  // slots whose neighbour joins the frontier (nb[s] then holds it)
        if (valid) {
            load_nb<W>(enc ? p.elle : p.ell, f, nb);
            heavy = nb[0] == kHeavy;
            if constexpr (MODE == kCount)
                if (p.count_te && !heavy) te_loc += row_edges<W>(nb, enc ? enc_vertex(f) : f);
            if (!heavy) {
#pragma unroll
                for (int s = 0; s < W; ++s) {
                    int w = nb[s];
                    bool fresh;
                    if (enc)
                        fresh = test_and_mark_enc(bm, nb[s], &w);
                    else
                        fresh = test_and_mark(bm, sm, w);
                    if (fresh) {
                        if (w < t0) {
                            newm |= 1u << s;
                            nb[s] = w;
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
            }
        }
        // the new frontier vertices, one per lane per round
        for (;;) {
            const bool has = newm != 0;
            const unsigned b = __ballot_sync(kFull, has);
            if (!b) break;
            int v = 0;
            if (has) {
                const int s0 = __ffs(newm) - 1;
                newm &= newm - 1;
#pragma unroll
                for (int s = 0; s < W; ++s)
                    if (s == s0) v = nb[s];
            }
            ring_append(h, has, b, v, ring, R, head, tail, spool, pcap, pool, pend, nspill);
        }
        // heavy vertices (degree > W): one warp each, over A's CSR row
        unsigned hm = __ballot_sync(kFull, valid && heavy);
        while (hm) {
            const int src = __ffs(hm) - 1;
            hm &= hm - 1;
            const int len = __shfl_sync(kFull, nb[1], src);
            const int64_t off =
                heavy_off(__shfl_sync(kFull, nb[2], src), __shfl_sync(kFull, nb[3], src));
            if (lane == 0) atomicAdd(&h.te, (unsigned long long)len);
            for (int eb = 0; eb < len; eb += 32) {
                const int e = eb + lane;
                bool fr = false;
                int w = -1;
                if (e < len) {
                    w = __ldg(p.ci + off + e);
                    if (test_and_mark(bm, sm, w)) {
                        if (w < t0) {
                            fr = true;
                        } else if (w > i) {
                            ++a.ucnt;
                            a.lmax = max(a.lmax, w);
                        }
                    }
                }
                const unsigned b = __ballot_sync(kFull, fr);
                if (b) ring_append(h, fr, b, w, ring, R, head, tail, spool, pcap, pool, pend, nspill);
            }
        }
        // the m expanded vertices leave the count, their children join it (one update;
        // children donated to the pool on the way were counted by ring_donate)
        if (lane == 0 && pend != m) atomicAdd(&h.outst, pend - m);
        pend = 0;
    }
    if (lane == 0) {
        atomicAdd(&h.sv, nproc);
        if (nspill) atomicAdd(&h.spills, nspill);
    }
    if (MODE == kCount && p.count_te) {
#pragma unroll
        for (int o = 16; o; o >>= 1) te_loc += __shfl_xor_sync(kFull, te_loc, o);
        if (lane == 0 && te_loc) atomicAdd(&h.te, te_loc);
    }
    __syncthreads();
    a.lmin = 0;  // marks somewhere below t0: clear from word 0 (summary walk)
}

// Level-synchronous BFS from threshold t0 over unvisited vertices < t0 (Alg. 1).
// Level lev reads queue lev&1 and writes queue (lev+1)&1 (shared, spilling to the CTA's two
// HBM halves); the level counters rotate through h.cnt[0..2] so one barrier per level suffices.
// Queue and spill addresses are recomputed from the launch parameters each level rather than
// carried in registers (at 32 registers per thread they would otherwise spill).
template <int NT, int W, int VIS, int MODE, bool ASYNC>
__device__ void bfs(const Fill2Params &p, Hdr &h, const VisMap<VIS> &bm, uint32_t *sm, int32_t *qA,
                    const int i, const int t0, RowAcc &a)
{
    if constexpr (ASYNC) {
        if (p.aring) {
            bfs_async<NT, W, VIS, MODE>(p, h, bm, sm, qA, i, t0, a);
            return;
        }
    }
    const int tid = threadIdx.x;
    if (tid == 0) {
        qA[0] = t0;
        h.cnt[1] = h.cnt[2] = 0;
        h.sv += 1;
    }
    __syncthreads();
    int fsize = 1, cur = 0;  // cur: counter index of the level being read
    for (int lev = 0;; ++lev) {
        const int par = lev & 1;
        const int nxt = cur == 2 ? 0 : cur + 1;
        int32_t *gA = p.gspill + (size_t)blockIdx.x * 2 * p.spill_cap;
        if (p.kloc)
            scan_level<NT, W, VIS, true, MODE>(p, h, bm, sm, qA + par * p.q, gA + par * p.spill_cap,
                                         fsize, &h.cnt[nxt], qA + (par ^ 1) * p.q,
                                         gA + (par ^ 1) * p.spill_cap, i, t0, a);
        else if (LUSYM_VPT > 1)
            scan_level_multi<NT, W, VIS, LUSYM_VPT>(p, h, bm, sm, qA + par * p.q,
                                                    gA + par * p.spill_cap, fsize, &h.cnt[nxt],
                                                    qA + (par ^ 1) * p.q,
                                                    gA + (par ^ 1) * p.spill_cap, i, t0, a);
        else
            scan_level<NT, W, VIS, false, MODE>(p, h, bm, sm, qA + par * p.q, gA + par * p.spill_cap,
                                          fsize, &h.cnt[nxt], qA + (par ^ 1) * p.q,
                                          gA + (par ^ 1) * p.spill_cap, i, t0, a);
        __syncthreads();
        fsize = h.cnt[nxt];
        if (fsize == 0) break;
        if (tid == 0) {
            h.cnt[cur] = 0;  // becomes the write counter two levels from now
            h.sv += fsize;
            if (fsize > p.q) h.spills += fsize - p.q;
        }
        cur = nxt;
    }
    a.lmin = 0;  // the BFS marked vertices somewhere below t0: clear from word 0 (summary walk)
}

// Kernel key -> CTA size and register budget.  KEY = NT (128..1024): registers for
// LUSYM_THREADS_PER_SM resident threads (32 per thread at 2048).  KEY = 1025: 1024 threads with
// the one-CTA-per-SM budget (64 registers, no spills) for classes whose shared memory already
// limits them to one CTA per SM (the planner picks it).
template <int KEY>
struct NtCfg {
    // (LUSYM_THREADS_PER_SM_SMALL: a separate budget for 64- and 128-thread CTAs; 1536, i.e.
    // ~40 registers, measured in session 2 against 2048: cfg2 +10%, cfg3 +6%, cfg1 +70%,
    // profiles/r02/ab_regs2.log, so both stay at 2048)
    static constexpr int NT = KEY,
                         MINB = (KEY <= 128 ? LUSYM_THREADS_PER_SM_SMALL : LUSYM_THREADS_PER_SM) / KEY;
};
template <>
struct NtCfg<1025> {
    static constexpr int NT = 1024, MINB = 1;
};

// MODE: kCount (symbolic_1, counts only), kStage (counts + rows staged into the HBM pool, so
// symbolic_2 becomes a placement copy), kEmit (symbolic_2 by traversal, into the final CSR).
template <int KEY, int W, int MODE, int VIS>
__global__ void __launch_bounds__(NtCfg<KEY>::NT, NtCfg<KEY>::MINB)
    fill2_kernel(const Fill2Params p)
{
    constexpr int NT = NtCfg<KEY>::NT;
    constexpr bool GB = VIS == kVisGlobal;
    extern __shared__ __align__(16) unsigned char smem[];
    Hdr &h = *reinterpret_cast<Hdr *>(smem);
    // shared layout: header | visited bitmap (at a constant offset, so the hot bit tests need
    // no address arithmetic beyond the word index) | summary | two frontier queues
    VisMap<VIS> bm;
    bm.g = p.gbitmap ? p.gbitmap + (size_t)blockIdx.x * p.gbitmap_stride : nullptr;
    bm.lbw = p.lbw;
    bm.nw = GB ? 0 : p.nw;
    uint32_t *sm;
    int32_t *qA, *qB;
    if constexpr (GB) {
        bm.s = nullptr;
        sm = reinterpret_cast<uint32_t *>(smem + kHdrBytes);
    } else {
        bm.s = reinterpret_cast<uint32_t *>(smem + kHdrBytes);
        sm = bm.s + p.nw;  // p.nw = shared visited words (whole swizzle groups)
    }
    bm.ssum = (uint32_t)__cvta_generic_to_shared(sm);
    qA = reinterpret_cast<int32_t *>(sm + p.sw);
    qB = qA + p.q;
    const int tid = threadIdx.x, lane = tid & 31;
    (void)lane;
    if constexpr (!GB) check_smem_base(smem);
    for (int w = tid; w < p.sw; w += NT) sm[w] = 0;
    if constexpr (!GB)
        for (int w = tid; w < p.nw; w += NT) bm.s[w] = 0;

    RowAcc a;
    if (tid == 0) h.te = h.sv = h.spills = 0;
    const int nrows = p.row_end - p.row_begin;
    for (;;) {
        if (tid == 0) {
            const unsigned long long c = atomicAdd(p.row_counter, 1ull);
            int r = -1;
            if (p.row_list) {
                const unsigned long long len =
                    p.list_len_dev ? *p.list_len_dev : (unsigned long long)p.list_len;
                if (c < len) r = p.row_list[c];
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
        const long long t_row = p.row_prof ? clock64() : 0;
        const unsigned long long sv_row = h.sv;  // read and written by thread 0 only
        int n_bfs = 0, n_win = 0;
#if LUSYM_PHASE_PROF  // diagnostic build: per-row cycles by phase of the threshold loop
        long long ph_col = 0, ph_win = 0, ph_bfs = 0, ph_t = 0;
#define PH_MARK(acc)                                         \
    do {                                                     \
        const long long ph_now = clock64();                  \
        if (ph_t) acc += ph_now - ph_t;                      \
        ph_t = ph_now;                                       \
    } while (0)
#else
#define PH_MARK(acc) do { } while (0)
#endif
        a.ucnt = 0;
        a.lmin = i;
        a.lmax = i;

        // ---- seed: fill(src) = src; for v in A(src,:) fill(v) = src  (L116-129)
        const int64_t rb = p.rp[i], re = p.rp[i + 1];
        for (int64_t k = rb + tid; k < re; k += NT) {
            const int v = __ldg(p.ci + k);
            mark(bm, sm, v);
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
        if (tid == 0) {
            mark(bm, sm, i);
            h.te += (unsigned long long)(re - rb);
        }
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
        // "done" marks (HBM slot of this CTA) of simple thresholds processed ahead of the pointer,
        // so a re-collected window skips them; non-simple ones are re-checked, in a window that
        // shrinks to kSmallWin after it was cut short and doubles back while it is consumed
        uint32_t *dm = p.dbitmap + (size_t)blockIdx.x * p.gbitmap_stride;
        bool dused = false;
        bool deferred = false;  // block-uniform
        int cap = p.wcap;
        // ---- thresholds in increasing order (L130)
        for (;;) {
            // the previous window's tns/newmin were read before its last barrier; collect ends
            // with a barrier, so this reset is visible before the window's atomicMin's
            if (tid == 0) {
                h.tns = INT_MAX;
                h.newmin = INT_MAX;
            }
            PH_MARK(ph_bfs);
            const int wc = collect<NT, VIS>(bm, sm, dused ? dm : nullptr, ptr + 1, i, qA, cap,
                                           h.scan);
            PH_MARK(ph_col);
            if (wc == 0) break;
            ++n_win;
            if constexpr (MODE != kEmit) {
                // reading G8: a row whose threshold chain is this long is abandoned here and
                // finished after the pass by the row-merge tail (block-uniform decision); in
                // kCount mode without a list (the planner's sample) it is just abandoned
                if (n_win == p.defer_win + 1 && p.defer_win > 0 && i >= p.defer_from) {
                    if (tid == 0) {
                        bool ok = true;
                        if (p.defer_list) {
                            const unsigned long long slot = atomicAdd(p.defer_cnt, 1ull);
                            ok = slot < (unsigned long long)p.defer_max;
                            if (ok) {
                                p.defer_list[slot] = i;
                                p.row_off[i] = kRowDeferred;
                            }
                        }
                        h.defer = ok;
                    }
                    __syncthreads();
                    if (h.defer) {
                        deferred = true;
                        break;
                    }
                }
            }
            int nm = INT_MAX;
            unsigned long long w_te = 0;  // traversed edges of this thread's done thresholds
            for (int base = 0; base < wc; base += NT) {
#if LUSYM_WARP_EXIT
                if (base + (tid & ~31) >= wc) break;  // warp-uniform, as in scan_level
#endif
                const int k = base + tid;
                const bool valid = k < wc;
                const int t = valid ? qA[k] : 0;
                int nb[ell_stride<W>()];
#pragma unroll
                for (int s = 0; s < ell_stride<W>(); ++s) nb[s] = 0;
                bool heavy = false, done = false;
                if (valid) {
                    load_nb<W>(p.ell, t, nb);
                    heavy = nb[0] == kHeavy;
                }
                if (valid && !heavy) {
                    bool simple = true;
#pragma unroll
                    for (int s = 0; s < W; ++s) {
                        const int w = nb[s];
                        if (w < t && !visited(bm, w)) simple = false;
                    }
                    if (!simple) {
                        atomicMin(&h.tns, t);
                    } else {
                        done = true;
                        if constexpr (MODE == kCount)
                            if (p.count_te) w_te += row_edges<W>(nb, t);
#pragma unroll
                        for (int s = 0; s < W; ++s) {
                            const int w = nb[s];
                            if (w > t && test_and_mark(bm, sm, w)) {
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
                        if (w < tt && !visited(bm, w)) ok = false;
                    }
                    ok = __all_sync(kFull, ok);
                    // a heavy threshold is scanned once: when it is simple here, else by its BFS
                    if (lane == 0 && ok) atomicAdd(&h.te, (unsigned long long)len);
                    if (lane == src) done = ok;
                    if (!ok) {
                        if (lane == 0) atomicMin(&h.tns, tt);
                    } else {
                        for (int e = lane; e < len; e += 32) {
                            const int w = __ldg(p.ci + off + e);
                            if (w > tt && test_and_mark(bm, sm, w)) {
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
                if (valid) qB[k] = done ? 1 : 0;
                // scanned vertices: a threshold counts once, when it is done here
                // (simple) or when its BFS starts (non-simple ones are re-collected until then)
                const unsigned db = __ballot_sync(kFull, valid && done);
                if (lane == 0 && db) atomicAdd(&h.sv, (unsigned long long)__popc(db));
            }
            if (MODE == kCount && p.count_te) {
#pragma unroll
                for (int o = 16; o; o >>= 1) w_te += __shfl_xor_sync(kFull, w_te, o);
                if (lane == 0 && w_te) atomicAdd(&h.te, w_te);
            }
            if (nm != INT_MAX) atomicMin(&h.newmin, nm);
            __syncthreads();
            // m = smallest pending threshold now: a non-simple candidate (tns) or a vertex just
            // marked by a simple one (newmin)
            const int tns = h.tns, newmin = h.newmin;
            const int m = min(tns, newmin);
            const int last = qA[wc - 1];
            const int nptr = m > last ? last : (m == tns ? m : m - 1);
            // every visited bit in (ptr, nptr] is an L entry now (no BFS has marked below m yet):
            // emit / count them in increasing order as the pointer passes (L122-143)
            if (nptr < last) {  // simple candidates beyond the pointer are finished: mark them
                for (int k = tid; k < wc; k += NT) {
                    const int t = qA[k];
                    if (t > nptr && qB[k]) atomicOr(dm + (t >> 5), 1u << (t & 31));
                }
                dused = true;
            }
            // the barriers inside emit_range order these marks (and the reads of qA/qB) before
            // the next collect and the BFS; an empty range has none, so add one
            Lcnt += emit_range<NT, VIS, MODE != kCount>(bm, sm, ptr + 1, nptr + 1, ldst, Lcnt, lcap,
                                                       h.scan);
            if (nptr <= ptr) __syncthreads();
            PH_MARK(ph_win);
            if (m <= last && m == tns) {  // smallest pending threshold: below-exploration
                bfs<NT, W, VIS, MODE, (KEY == 1025)>(p, h, bm, sm, qA, i, m, a);
                ++n_bfs;
            }
            cap = m <= last ? min(cap, kSmallWin) : min(2 * cap, p.wcap);
            ptr = nptr;
        }
        // thresholds finished ahead of the pointer and never re-collected: the rest of (ptr, i)
        if (!deferred)
            Lcnt += emit_range<NT, VIS, MODE != kCount>(bm, sm, ptr + 1, i, ldst, Lcnt, lcap,
                                                       h.scan);
        if (dused)  // leave the done map zero for the next row
            for (int w = (h.minseed >> 5) + tid; w <= ((i - 1) >> 5); w += NT) dm[w] = 0;

        // ---- U part, diagonal, count / emission
        if (a.ucnt) atomicAdd(&h.ucnt, a.ucnt);
        if (a.lmin < i) atomicMin(&h.lmin, a.lmin);
        if (a.lmax > i) atomicMax(&h.lmax, a.lmax);
        __syncthreads();
        const int ucnt = h.ucnt, diag = h.diag, gmin = h.lmin, gmax = h.lmax;
        const int len = Lcnt + diag + ucnt;
        if constexpr (MODE == kCount) {
            if (tid == 0 && !deferred) p.fill_count[i] = len;
        } else if constexpr (MODE == kStage) {
          if (!deferred) {
            // reserve len entries of the pool; rows that do not fit are re-traversed by emit
            if (tid == 0) {
                p.fill_count[i] = len;
                p.ucut[i] = Lcnt + diag;
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
                emit_range<NT, VIS, true>(bm, sm, i + 1, gmax + 1, dst + Lcnt + diag, 0, INT64_MAX,
                                         h.scan);
            }
          }
        } else {
            if (lcap != (int64_t)len) {
                if (tid == 0) atomicAdd(p.stats + kStatErr, 1ull);
            } else {
                if (diag && tid == 0) ldst[Lcnt] = i;
                emit_range<NT, VIS, true>(bm, sm, i + 1, gmax + 1, ldst + Lcnt + diag, 0, INT64_MAX,
                                         h.scan);
            }
        }
        if (p.row_prof && tid == 0) {
            p.row_prof[4 * (size_t)i + 0] = clock64() - t_row;
#if LUSYM_PHASE_PROF
            p.row_prof[4 * (size_t)i + 1] = ph_col;
            p.row_prof[4 * (size_t)i + 2] = ph_win;
            p.row_prof[4 * (size_t)i + 3] = ph_bfs;
            (void)n_bfs;
            (void)n_win;
            (void)sv_row;
#else
            p.row_prof[4 * (size_t)i + 1] = (long long)(h.sv - sv_row);
            p.row_prof[4 * (size_t)i + 2] = n_bfs;
            p.row_prof[4 * (size_t)i + 3] = n_win;
#endif
        }
        // ---- clear the dirty word range (fill(:) = 0 for the next row, L115)
        clear_words<NT, VIS>(bm, sm, gmin >> 5, gmax >> 5);
        __syncthreads();
    }

    // flush statistics (every heavy-vertex atomic finished before the last barrier)
    if (tid == 0) {
        atomicAdd(p.stats + kStatEdges, h.te);
        atomicAdd(p.stats + kStatVerts, h.sv);
        if (h.spills) atomicAdd(p.stats + kStatSpills, h.spills);
    }
}

template <int NT, int W, int VIS>
cudaError_t launch_w_vis(const Fill2Params &p, int mode, int grid, size_t smem, cudaStream_t s)
{
    constexpr int B = NtCfg<NT>::NT;  // NT here is the kernel key
    if (mode == kCount)
        fill2_kernel<NT, W, kCount, VIS><<<grid, B, smem, s>>>(p);
    else if (mode == kStage)
        fill2_kernel<NT, W, kStage, VIS><<<grid, B, smem, s>>>(p);
    else
        fill2_kernel<NT, W, kEmit, VIS><<<grid, B, smem, s>>>(p);
    return cudaGetLastError();
}

template <int NT, int W, int VIS>
cudaError_t configure_w_vis(size_t smem)
{
    const void *fns[3] = {(const void *)fill2_kernel<NT, W, kCount, VIS>,
                          (const void *)fill2_kernel<NT, W, kStage, VIS>,
                          (const void *)fill2_kernel<NT, W, kEmit, VIS>};
    for (const void *f : fns) {
        cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
        cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    }
    return cudaSuccess;
}

template <int NT, int W, int VIS>
cudaError_t occupancy_w_vis(size_t smem, int *occ)
{
    const void *fns[3] = {(const void *)fill2_kernel<NT, W, kCount, VIS>,
                          (const void *)fill2_kernel<NT, W, kStage, VIS>,
                          (const void *)fill2_kernel<NT, W, kEmit, VIS>};
    int best = 1 << 30;
    for (const void *f : fns) {
        int o = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, f, NtCfg<NT>::NT, smem);
        if (e != cudaSuccess) return e;
        best = o < best ? o : best;
    }
    *occ = best;
    return cudaSuccess;
}

template <int NT, template <int, int, int> class Op, class... Args>
cudaError_t dispatch_w_vis(int w, int vis, Args... args)
{
    if (w == 4 && vis == kVisSmem) return Op<NT, 4, kVisSmem>::run(args...);
    if (w == 4 && vis == kVisGlobal) return Op<NT, 4, kVisGlobal>::run(args...);
    if (w == 4 && vis == kVisSplit) return Op<NT, 4, kVisSplit>::run(args...);
    if (w == 6 && vis == kVisSmem) return Op<NT, 6, kVisSmem>::run(args...);
    if (w == 6 && vis == kVisGlobal) return Op<NT, 6, kVisGlobal>::run(args...);
    if (w == 6 && vis == kVisSplit) return Op<NT, 6, kVisSplit>::run(args...);
    if (w == 8 && vis == kVisSmem) return Op<NT, 8, kVisSmem>::run(args...);
    if (w == 8 && vis == kVisGlobal) return Op<NT, 8, kVisGlobal>::run(args...);
    if (w == 8 && vis == kVisSplit) return Op<NT, 8, kVisSplit>::run(args...);
    return cudaErrorInvalidValue;
}

template <int NT, int W, int VIS>
struct LaunchOp {
    static cudaError_t run(const Fill2Params *p, int mode, int grid, size_t smem, cudaStream_t s)
    {
        return launch_w_vis<NT, W, VIS>(*p, mode, grid, smem, s);
    }
};
template <int NT, int W, int VIS>
struct ConfigOp {
    static cudaError_t run(size_t smem) { return configure_w_vis<NT, W, VIS>(smem); }
};
template <int NT, int W, int VIS>
struct OccOp {
    static cudaError_t run(size_t smem, int *occ) { return occupancy_w_vis<NT, W, VIS>(smem, occ); }
};

}  // namespace f2

// Explicit per-NT entry points (one translation unit per CTA size: fill2_nt<NT>.cu).
#define LUSYM_F2_INSTANTIATE(NTV)                                                            \
    template <>                                                                              \
    cudaError_t fill2_launch_nt<NTV>(const Fill2Params &p, int w, int mode, int vis,         \
                                     int grid, size_t smem, cudaStream_t s)                  \
    {                                                                                        \
        return f2::dispatch_w_vis<NTV, f2::LaunchOp>(w, vis, &p, mode, grid, smem, s);       \
    }                                                                                        \
    template <>                                                                              \
    cudaError_t fill2_configure_nt<NTV>(int w, int vis, size_t smem)                         \
    {                                                                                        \
        return f2::dispatch_w_vis<NTV, f2::ConfigOp>(w, vis, smem);                          \
    }                                                                                        \
    template <>                                                                              \
    cudaError_t fill2_occupancy_nt<NTV>(int w, int vis, size_t smem, int *occ)               \
    {                                                                                        \
        return f2::dispatch_w_vis<NTV, f2::OccOp>(w, vis, smem, occ);                        \
    }

}  // namespace lusym
