// Comparer ("compare" kernel, M8 + M9) for sm_100a -- two implementations.
//
// Paper: Listing 1.  For each locus i and each selected strand the kernel
// walks the non-N query positions (comp_index, -1-terminated), counts genome
// bases outside the query letter's IUPAC set, stops early once the count
// exceeds the threshold and, if the count is <= threshold,
// appends (count, direction, locus) through an atomic counter.
// The '-' half compares the reverse-complemented query against the same '+' window
// (P:L231-L236).  The query table is staged in local (shared) memory (the
// paper's opt3).  This kernel is ~98% of kernel time.
//
// v1 "popc"  (cof_comparer_popc): items in registers (R per thread), guide records in
//   shared memory; per (item, guide) mm = popc(care & ((w_lo^g_lo) | (w_hi^g_hi) | w_nm))
//   with the window pre-masked by the group's care mask -> 2 LOP3 + POPC + IADD.  Bound by
//   the quarter-rate POPC pipe (16/clk/SM measured on B200, tools/microbench_pipes.cu).
// v2 "table" (cof_comparer_table): bit-sliced over 32 guides.  For each position pair of
//   an item, one 64-bit shared-memory lookup indexed by the pair's two genome bases returns
//   the 2-bit mismatch count of all 32 guides of a block (bit k = guide k); a LOP3
//   carry-save adder tree sums the pairs and a borrow chain against the bit-sliced
//   thresholds yields the 32-guide hit mask.  No POPC, ~1.3 ALU ops + 0.3 LDS per
//   comparison.  Handles any IUPAC guide letter and per-guide thresholds uniformly.
#include <algorithm>

#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"
#include "csa_gen.cuh"

namespace cof {

constexpr int CT = 256;   // threads per CTA
constexpr uint64_t ON_DEVICE = COF_COUNT_ON_DEVICE;
constexpr uint32_t MAX_TABLE_BLOCKS = 128;   // 4096 guides per launch of the table comparer
constexpr uint32_t FUSED_MAX_TICKETS = 1024; // grab counters (one per fused launch) after the finder workspace

// Window word of the table comparer: one 32-bit slice, or 64 bits when the compared span
// exceeds 32 positions (L > 32).
template <bool W64> struct WinSel { using T = uint32_t; };
template <> struct WinSel<true> { using T = unsigned long long; };
template <bool W64> using WinT = typename WinSel<W64>::T;

struct CompareArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    const uint32_t* items[2];
    uint64_t n[2];                 // ON_DEVICE: read counters[0..1]
    uint64_t items_cap;
    unsigned long long* hits;
    uint64_t cap;
    unsigned long long* counters;  // [0] n_fwd [1] n_rev [2] n_hits
    // v1
    const uint4* groups[2];        // GroupDesc as uint4
    const uint4* recs[2];
    uint32_t n_groups, n_recs;
};

__device__ __forceinline__ void item_counts(const CompareArgs& a, uint64_t& n0, uint64_t& n1) {
    n0 = a.n[0] == ON_DEVICE ? (uint64_t)a.counters[0] : a.n[0];
    n1 = a.n[1] == ON_DEVICE ? (uint64_t)a.counters[1] : a.n[1];
    if (n0 > a.items_cap) n0 = a.items_cap;
    if (n1 > a.items_cap) n1 = a.items_cap;
}

// Warp-aggregated append of one key per predicated lane (old = atomic_inc(entrycount)).
__device__ __forceinline__ void emit(const CompareArgs& a, bool pred, unsigned long long key) {
    const unsigned act = __activemask();
    const unsigned m = __ballot_sync(act, pred);
    if (!pred) return;
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(m) - 1;
    unsigned long long base = 0;
    if (lane == leader) base = atomicAdd(&a.counters[2], (unsigned long long)__popc(m));
    base = __shfl_sync(m, base, leader);
    const unsigned long long o = base + __popc(m & lanemask_lt());
    if (o < a.cap) a.hits[o] = key;
}

__device__ __forceinline__ unsigned long long hit_key(uint32_t pos, uint32_t strand, uint32_t guide, uint32_t mm) {
    return ((unsigned long long)pos << 32) | ((unsigned long long)strand << 31) |
           ((unsigned long long)guide << 7) | (unsigned long long)mm;
}

// ============================================================================ v1 popc
template <int R, bool SMEM>
__global__ void __launch_bounds__(CT) cof_comparer_popc(const __grid_constant__ CompareArgs a) {
    extern __shared__ __align__(16) uint4 s_tab[];
    const uint4* G[2];
    const uint4* Rc[2];
    if (SMEM) {
        const uint32_t ng = a.n_groups, nr = a.n_recs;
        for (uint32_t i = threadIdx.x; i < ng; i += CT) {
            s_tab[i] = a.groups[0][i];
            s_tab[ng + i] = a.groups[1][i];
        }
        for (uint32_t i = threadIdx.x; i < nr; i += CT) {
            s_tab[2 * ng + i] = a.recs[0][i];
            s_tab[2 * ng + nr + i] = a.recs[1][i];
        }
        __syncthreads();
        G[0] = s_tab; G[1] = s_tab + ng; Rc[0] = s_tab + 2 * ng; Rc[1] = s_tab + 2 * ng + nr;
    } else {
        G[0] = a.groups[0]; G[1] = a.groups[1]; Rc[0] = a.recs[0]; Rc[1] = a.recs[1];
    }
    uint64_t n0, n1;
    item_counts(a, n0, n1);
    const uint64_t per_tile = (uint64_t)CT * R;
    const uint64_t t0 = (n0 + per_tile - 1) / per_tile, t1 = (n1 + per_tile - 1) / per_tile;
    for (uint64_t tile = blockIdx.x; tile < t0 + t1; tile += gridDim.x) {
        const uint32_t st = tile < t0 ? 0u : 1u;
        const uint64_t base = (st == 0 ? tile : tile - t0) * per_tile;
        const uint64_t nst = st == 0 ? n0 : n1;
        uint32_t pos[R], wl[R], wh[R], wn[R];
        bool ok[R];
#pragma unroll
        for (int r = 0; r < R; r++) {
            const uint64_t idx = base + (uint64_t)r * CT + threadIdx.x;
            ok[r] = idx < nst;
            pos[r] = ok[r] ? __ldg(a.items[st] + idx) : 0u;
            wl[r] = plane_window(a.lo, pos[r]);
            wh[r] = plane_window(a.hi, pos[r]);
            wn[r] = plane_window(a.nm, pos[r]);
        }
        for (uint32_t g = 0; g < a.n_groups; g++) {
            const uint4 gd = G[st][g];             // {care, kind, rec_begin, n_guides}
            const uint32_t care = gd.x;
            if (gd.y == GROUP_CONCRETE) {
                uint32_t ml[R], mh[R], mn[R];
#pragma unroll
                for (int r = 0; r < R; r++) { ml[r] = wl[r] & care; mh[r] = wh[r] & care; mn[r] = wn[r] & care; }
                const uint4* rec = Rc[st] + gd.z;
                for (uint32_t k = 0; k < gd.w; k++) {
                    const uint4 q = rec[k];       // {g_lo, g_hi, -(t+1), guide}
                    int32_t any = 0;
#pragma unroll
                    for (int r = 0; r < R; r++) {
                        const uint32_t y = ((ml[r] ^ q.x) | mn[r]) | (mh[r] ^ q.y);
                        any |= __popc(y) + (int32_t)q.z;
                    }
                    if (any < 0) {
#pragma unroll
                        for (int r = 0; r < R; r++) {
                            const uint32_t y = ((ml[r] ^ q.x) | mn[r]) | (mh[r] ^ q.y);
                            const uint32_t mm = (uint32_t)__popc(y);
                            emit(a, ok[r] && (int32_t)mm + (int32_t)q.z < 0, hit_key(pos[r], st, q.w, mm));
                        }
                    }
                }
            } else {
                // degenerate guide letters: one-hot window planes, match = OR_b (is_b & guide_b)
                uint32_t isA[R], isC[R], isG[R], isT[R];
#pragma unroll
                for (int r = 0; r < R; r++) {
                    isA[r] = ~wl[r] & ~wh[r] & ~wn[r];
                    isC[r] = wl[r] & ~wh[r] & ~wn[r];
                    isG[r] = ~wl[r] & wh[r] & ~wn[r];
                    isT[r] = wl[r] & wh[r] & ~wn[r];
                }
                const uint4* rec = Rc[st] + gd.z;
                for (uint32_t k = 0; k < gd.w; k++) {
                    const uint4 q = rec[2 * k];        // one-hot {A, C, G, T}
                    const uint4 q2 = rec[2 * k + 1];   // {care, -(t+1), guide, 0}
#pragma unroll
                    for (int r = 0; r < R; r++) {
                        const uint32_t match = (isA[r] & q.x) | (isC[r] & q.y) | (isG[r] & q.z) | (isT[r] & q.w);
                        const uint32_t mm = (uint32_t)__popc(q2.x & ~match);
                        emit(a, ok[r] && (int32_t)mm + (int32_t)q2.y < 0, hit_key(pos[r], st, q2.z, mm));
                    }
                }
            }
        }
    }
}

// ============================================================================ v2 table
// Shared-memory addressing of the pair tables: the entry of pair q for bases (b1, b2) of an
// item is read at base[q] + OFF + q * 128, where OFF = the guide block's table offset and
// q * 128 (pair q's 16 ACGT entries) are compile-time immediates of the LDS; base[q] is the
// 128-byte-aligned table base plus the entry's offset relative to q * 128.
// (wl, wh, wn: windows starting at window offset pl.p0, the first compared position;
// WT = uint32_t, or unsigned long long for compared spans > 32 (two-word windows, L > 32))
template <int NP, typename WT>
__device__ __forceinline__ void pair_offsets(const PairLayout& pl, uint32_t s_base, WT wl, WT wh,
                                             WT wn, uint32_t (&base)[NP]) {
#pragma unroll
    for (int q = 0; q < NP; q++) {
        const uint32_t j1 = pl.j1[q] - pl.p0, j2 = pl.j2[q] >= 0xFEu ? 0xFFu : pl.j2[q] - pl.p0;
        const uint32_t b1 = ((wn >> j1) & 1u) ? 4u : (uint32_t)(((wl >> j1) & 1u) | (((wh >> j1) & 1u) << 1));
        uint32_t b2 = 0;
        if (j2 < 64u) b2 = ((wn >> j2) & 1u) ? 4u : (uint32_t)(((wl >> j2) & 1u) | (((wh >> j2) & 1u) << 1));
        base[q] = s_base + pair_entry(NP, (uint32_t)q, b1, b2) * 8u - (uint32_t)q * 128u;
    }
}

template <uint32_t OFF>
__device__ __forceinline__ void lds64(uint32_t addr, uint32_t& x, uint32_t& y) {
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2+%3];" : "=r"(x), "=r"(y) : "r"(addr), "n"(OFF));
}

// The NP pair-entry loads of one item and guide block: pair q at base[q] + OFF + q * 128.
template <int NP, uint32_t OFF, int Q = 0>
__device__ __forceinline__ void lds_pairs(const uint32_t (&base)[NP], uint32_t (&v0)[NP], uint32_t (&v1)[NP]) {
    if constexpr (Q < NP) {
        lds64<OFF + (uint32_t)Q * 128u>(base[Q], v0[Q], v1[Q]);
        lds_pairs<NP, OFF, Q + 1>(base, v0, v1);
    }
}

// Arguments of one table-comparer launch: ONE strand, up to MAX_TABLE_BLOCKS guide blocks.
struct TableArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    const uint32_t* items;
    uint64_t n;                    // ON_DEVICE: read counters[strand]
    uint64_t items_cap;
    unsigned long long* hits;
    uint64_t cap;
    unsigned long long* counters;  // [0] n_fwd [1] n_rev [2] n_hits
    const uint2* ptab;             // [n_blocks][NP][25] of this strand, first block = block_base
    uint32_t strand;
    uint32_t n_blocks;
    uint32_t block_base;
    uint32_t blocks_per_chunk;     // guide blocks resident in shared memory at a time
    PairLayout pairs;
    uint32_t meta[MAX_TABLE_BLOCKS][8];   // per block: T0..T5 threshold planes, valid mask
    // fused find+compare: the finder's PAM masks replace the item list
    const uint4* masks;            // one {fwd0, rev0, fwd1, rev1} per word pair
    uint64_t n_wp;
    unsigned int* ticket;          // dynamic grab counter (zeroed per launch)
    uint32_t grab_rounds;          // FGRAB-word-pair ranges per ticket
};

// Hit mask (bit k = guide k of the block) of one item against one 32-guide block whose
// table starts OFF bytes past the item's base addresses.
// TC >= 0: every guide of the launch has threshold TC (compile-time constant: the borrow
// chain folds to a couple of LOP3); TC < 0: per-guide thresholds from the bit planes.
template <int NP, uint32_t OFF, int TC>
__device__ __forceinline__ uint32_t table_hits(const uint32_t (&base)[NP], const uint32_t* __restrict__ T,
                                               uint32_t (&s)[6]) {
    uint32_t v0[NP], v1[NP];
    lds_pairs<NP, OFF>(base, v0, v1);
    if constexpr (TC >= 0) {
        const uint32_t Tl[6] = {0u - (TC & 1u), 0u - ((TC >> 1) & 1u), 0u - ((TC >> 2) & 1u),
                                0u - ((TC >> 3) & 1u), 0u - ((TC >> 4) & 1u), 0u - ((TC >> 5) & 1u)};
        return csa_hits<NP>(v0, v1, Tl, T[6], s);
    } else {
        const uint32_t Tl[6] = {T[0], T[1], T[2], T[3], T[4], T[5]};
        return csa_hits<NP>(v0, v1, Tl, T[6], s);
    }
}

__device__ __noinline__ void table_emit_v(const TableArgs& a, const uint32_t* pos_ptr, uint32_t hitm, uint32_t s0,
                                          uint32_t s1, uint32_t s2, uint32_t s3, uint32_t s4, uint32_t s5,
                                          uint32_t guide0) {
    // Warp-aggregated append (P:L226 `old = atomic_inc(entrycount)` once per WARP and round):
    // every lane that reached here holds >= 1 hit; each round, every lane with hits left
    // emits one key, and one elected lane reserves the round's slots with a single atomic.
    const uint32_t pos = *pos_ptr;   // item list (global) or the fused kernel's queue (shared)
    const unsigned act = __activemask();
    const int lane = threadIdx.x & 31;
    for (;;) {
        const unsigned m = __ballot_sync(act, hitm != 0u);
        if (!m) break;
        const int leader = __ffs(m) - 1;
        unsigned long long base = 0;
        if (lane == leader) base = atomicAdd(&a.counters[2], (unsigned long long)__popc(m));
        base = __shfl_sync(act, base, leader);
        if (hitm) {
            const int k = __ffs(hitm) - 1;
            hitm &= hitm - 1;
            const uint32_t mm = ((s0 >> k) & 1u) | (((s1 >> k) & 1u) << 1) | (((s2 >> k) & 1u) << 2) |
                                (((s3 >> k) & 1u) << 3) | (((s4 >> k) & 1u) << 4) | (((s5 >> k) & 1u) << 5);
            const unsigned long long o = base + (unsigned)__popc(m & lanemask_lt());
            if (o < a.cap) a.hits[o] = hit_key(pos, a.strand, guide0 + (uint32_t)k, mm);
        }
    }
}

__device__ __forceinline__ void table_emit(const TableArgs& a, const uint32_t* pos_ptr, uint32_t hitm,
                                           const uint32_t (&s)[6], uint32_t guide0) {
    table_emit_v(a, pos_ptr, hitm, s[0], s[1], s[2], s[3], s[4], s[5], guide0);
}

// All resident blocks [0, nb) for the R items of this thread.  base[r][q] = shared address of
// item r's pair-q entry in block 0; groups of 4 blocks use immediate offsets.
template <int NP, int R, bool TAIL, int TC, int STRIDE = CT>
__device__ __forceinline__ void table_blocks(const TableArgs& a, uint32_t (&base)[R][NP], uint32_t nb, uint32_t gb0,
                                             const uint32_t* pos0, const uint32_t (&okm)[R]) {
    constexpr uint32_t BS = NP * 25 * 8;
    uint32_t b = 0;
    for (; b + 4 <= nb; b += 4) {
        const uint32_t* m = a.meta[gb0 + b];
#pragma unroll
        for (int r = 0; r < R; r++) {
            uint32_t sx[6];
            uint32_t h0 = table_hits<NP, 0 * BS, TC>(base[r], m + 0, sx);
            uint32_t h1 = table_hits<NP, 1 * BS, TC>(base[r], m + 8, sx);
            uint32_t h2 = table_hits<NP, 2 * BS, TC>(base[r], m + 16, sx);
            uint32_t h3 = table_hits<NP, 3 * BS, TC>(base[r], m + 24, sx);
            if (TAIL) { h0 &= okm[r]; h1 &= okm[r]; h2 &= okm[r]; h3 &= okm[r]; }
            if (h0 | h1 | h2 | h3) {          // rare: ~1 hit per 2.5e4 comparisons at t = 6
                // recompute the sums of the blocks that hit (keeps them out of the hot registers)
                const uint32_t* idx = pos0 + r * STRIDE;
                const uint32_t g0 = (a.block_base + gb0 + b) * 32u;
                uint32_t sh[6];
                if (h0) { table_hits<NP, 0 * BS, TC>(base[r], m + 0, sh); table_emit(a, idx, h0, sh, g0); }
                if (h1) { table_hits<NP, 1 * BS, TC>(base[r], m + 8, sh); table_emit(a, idx, h1, sh, g0 + 32u); }
                if (h2) { table_hits<NP, 2 * BS, TC>(base[r], m + 16, sh); table_emit(a, idx, h2, sh, g0 + 64u); }
                if (h3) { table_hits<NP, 3 * BS, TC>(base[r], m + 24, sh); table_emit(a, idx, h3, sh, g0 + 96u); }
            }
            if (b + 4 < nb) {
#pragma unroll
                for (int q = 0; q < NP; q++) base[r][q] += 4 * BS;
            }
        }
    }
    for (; b < nb; b++) {
        const uint32_t* m = a.meta[gb0 + b];
#pragma unroll
        for (int r = 0; r < R; r++) {
            uint32_t s0[6];
            uint32_t h0 = table_hits<NP, 0, TC>(base[r], m, s0);
            if (TAIL) h0 &= okm[r];
            if (h0) table_emit(a, pos0 + r * STRIDE, h0, s0, (a.block_base + gb0 + b) * 32u);
            if (b + 1 < nb) {
#pragma unroll
                for (int q = 0; q < NP; q++) base[r][q] += BS;
            }
        }
    }
}

// Table addresses (see pair_offsets) of the NP pair entries of one item, from its plane
// windows taken at pos + pairs.p0 (every compared offset is >= p0 and < p0 + 32, or
// < p0 + 64 with W64 windows).
template <int NP, bool W64>
__device__ __forceinline__ void window_bases(const PairLayout& pl, uint32_t s_base, WinT<W64> wl, WinT<W64> wh,
                                             WinT<W64> wn, uint32_t (&base)[NP]) {
    using WT = WinT<W64>;
    constexpr WT M33 = (WT)0x3333333333333333ull, MCC = (WT)0xCCCCCCCCCCCCCCCCull;
    if (pl.contig) {
        // fast path: with no N among the contiguous compared positions every pair index is
        // one nibble of Y (even pairs) or Z (odd pairs); s_base is 128-aligned, so the
        // entry offset ORs in (one SHF + one LOP3 per pair)
        const WT cm = pl.n_cmp >= 8 * sizeof(WT) ? ~(WT)0 : (((WT)1 << pl.n_cmp) - (WT)1);
        if ((wn & cm) == 0) {
            const WT Y = (wl & M33) | ((wh & M33) << 2);
            const WT Z = ((wl >> 2) & M33) | (wh & MCC);
#pragma unroll
            for (int q = 0; q < NP; q++) {
                const WT src = (q & 1) ? Z : Y;
                const int k = q >> 1;
                const uint32_t nib8 = (uint32_t)(k == 0 ? (src << 3) & 0x78u : (src >> (4 * k - 3)) & 0x78u);
                base[q] = s_base | nib8;
            }
            return;
        }
    }
    pair_offsets<NP, WT>(pl, s_base, wl, wh, wn, base);
}

// 64 consecutive bases from position p (bit j = base p+j): three plane words.
__device__ __forceinline__ unsigned long long plane_window64(const uint32_t* __restrict__ plane, uint32_t p) {
    const uint32_t w = p >> 5, sh = p & 31;
    const uint32_t x = __ldg(plane + w), y = __ldg(plane + w + 1), z = __ldg(plane + w + 2);
    return (unsigned long long)__funnelshift_r(x, y, sh) | ((unsigned long long)__funnelshift_r(y, z, sh) << 32);
}

template <bool W64>
__device__ __forceinline__ WinT<W64> item_window(const uint32_t* __restrict__ plane, uint32_t p) {
    if constexpr (W64) return plane_window64(plane, p);
    else return plane_window(plane, p);
}

template <int NP, bool W64>
__device__ __forceinline__ void item_bases(const TableArgs& a, uint32_t s_base, uint32_t pos, uint32_t (&base)[NP]) {
    const uint32_t p = pos + a.pairs.p0;
    window_bases<NP, W64>(a.pairs, s_base, item_window<W64>(a.lo, p), item_window<W64>(a.hi, p),
                          item_window<W64>(a.nm, p), base);
}

// Window prefetch of the table comparer: the plane words (lo, hi, nm; two each, three for
// W64 windows) an item's window needs are copied into this thread's shared-memory slots
// with cp.async one tile ahead, so the dependent global loads of the next tile overlap
// this tile's table work.  Slot k of thread t lives at word k * CT + t (conflict-free).
template <bool W64>
__device__ __forceinline__ void prefetch_window(const TableArgs& a, uint32_t slot, uint32_t pos) {
    constexpr uint32_t NWW = W64 ? 3 : 2;   // words per plane
    const uint32_t w = (pos + a.pairs.p0) >> 5;
#pragma unroll
    for (uint32_t k = 0; k < NWW; k++) {
        cp_async4(slot + (0 * NWW + k) * CT * 4, a.lo + w + k);
        cp_async4(slot + (1 * NWW + k) * CT * 4, a.hi + w + k);
        cp_async4(slot + (2 * NWW + k) * CT * 4, a.nm + w + k);
    }
}

template <bool W64>
__device__ __forceinline__ WinT<W64> slot_window(const uint32_t* slot, uint32_t sh) {
    if constexpr (W64)
        return (unsigned long long)__funnelshift_r(slot[0], slot[CT], sh) |
               ((unsigned long long)__funnelshift_r(slot[CT], slot[2 * CT], sh) << 32);
    else return __funnelshift_r(slot[0], slot[CT], sh);
}

template <int NP, bool W64>
__device__ __forceinline__ void slot_bases(const TableArgs& a, uint32_t s_base, const uint32_t* slot, uint32_t sh,
                                           uint32_t (&base)[NP]) {
    constexpr uint32_t NWW = W64 ? 3 : 2;
    window_bases<NP, W64>(a.pairs, s_base, slot_window<W64>(slot, sh), slot_window<W64>(slot + NWW * CT, sh),
                          slot_window<W64>(slot + 2 * NWW * CT, sh), base);
}

template <int NP, int R, int TC, bool W64>
__global__ void __launch_bounds__(CT, W64 ? 2 : 3) cof_comparer_table(const __grid_constant__ TableArgs a) {
    constexpr uint32_t NSLOT = W64 ? 9 : 6;   // prefetched plane words per item
    extern __shared__ __align__(16) uint8_t s_raw[];
    // shared: [blocks_per_chunk][NP][25] uint2 pair table of the resident chunk of blocks
    // (at the first 128-byte boundary), then the window slots
    constexpr uint32_t BS = NP * 25 * 8;
    const uint32_t s_raw_a = smem_u32(s_raw);
    const uint32_t s_base = (s_raw_a + 127u) & ~127u;
    uint2* s_tab_p = reinterpret_cast<uint2*>(s_raw + (s_base - s_raw_a));
    uint64_t n64 = a.n == ON_DEVICE ? (uint64_t)a.counters[a.strand] : a.n;
    if (n64 > a.items_cap) n64 = a.items_cap;
    // item indices fit 32 bits (n_bases < 2^32, checked by the host); an index past n that
    // wraps in the look-ahead below lands inside the list and is never consumed
    const uint32_t n = (uint32_t)n64;
    constexpr uint32_t per_tile = (uint32_t)CT * R;
    const uint32_t n_tiles = (uint32_t)((n64 + per_tile - 1) / per_tile);
    const uint32_t bpc = a.blocks_per_chunk;
    const uint32_t n_chunks = (a.n_blocks + bpc - 1) / bpc;
    uint32_t loaded = 0xFFFFFFFFu;

    // Two-stage prefetch: positions two tiles ahead (registers), plane words one tile ahead
    // (cp.async into per-thread shared slots after the resident table chunk).
    const uint32_t slot_off = (s_base - s_raw_a) + ((bpc * BS + 15u) & ~15u);
    const uint32_t slot_b = s_raw_a + slot_off;
    const uint32_t* slot_p = reinterpret_cast<const uint32_t*>(s_raw + slot_off);
    const uint32_t stride = gridDim.x * per_tile;
    uint32_t pos_next[R], shf[R];   // shf: window shift of the item whose words are in flight
    {
        const uint32_t i0 = blockIdx.x * per_tile + threadIdx.x;
#pragma unroll
        for (int r = 0; r < R; r++) {
            const uint32_t idx = i0 + (uint32_t)r * CT;
            const uint32_t p = idx < n ? __ldg(a.items + idx) : 0u;
            prefetch_window<W64>(a, slot_b + (uint32_t)(r * NSLOT * CT + threadIdx.x) * 4u, p);
            shf[r] = (p + a.pairs.p0) & 31u;
            pos_next[r] = (idx + stride) < n ? __ldg(a.items + idx + stride) : 0u;
        }
        cp_async_commit();
    }
    for (uint32_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const uint32_t t0 = tile * per_tile;
        const uint32_t item0 = t0 + threadIdx.x;
        const bool tail = n - t0 < per_tile;
        uint32_t base[R][NP], okm[R];
        cp_async_wait_all();
#pragma unroll
        for (int r = 0; r < R; r++) {
            const uint32_t idx = item0 + (uint32_t)r * CT;
            okm[r] = idx < n ? ~0u : 0u;
            slot_bases<NP, W64>(a, s_base, slot_p + r * NSLOT * CT + threadIdx.x, shf[r], base[r]);
        }
        // refill the slots for the next tile, then fetch the positions of the one after
#pragma unroll
        for (int r = 0; r < R; r++) {
            prefetch_window<W64>(a, slot_b + (uint32_t)(r * NSLOT * CT + threadIdx.x) * 4u, pos_next[r]);
            shf[r] = (pos_next[r] + a.pairs.p0) & 31u;
            const uint32_t nidx = item0 + 2 * stride + (uint32_t)r * CT;
            pos_next[r] = nidx < n ? __ldg(a.items + nidx) : 0u;
        }
        cp_async_commit();
        for (uint32_t ch = 0; ch < n_chunks; ch++) {
            const uint32_t b0 = ch * bpc;
            const uint32_t nb = min(bpc, a.n_blocks - b0);
            if (loaded != ch) {
                __syncthreads();
                const uint2* src = a.ptab + (size_t)b0 * NP * 25;
                const uint32_t n8 = nb * NP * 25;
                for (uint32_t i = threadIdx.x; i < n8; i += CT) s_tab_p[i] = __ldg(src + i);
                __syncthreads();
                loaded = ch;
            }
            if (tail) table_blocks<NP, R, true, TC>(a, base, nb, b0, a.items + item0, okm);
            else table_blocks<NP, R, false, TC>(a, base, nb, b0, a.items + item0, okm);
            if (n_chunks > 1) {
                // undo table_blocks' block-to-block advance (see its increments)
                const uint32_t inc = (nb & 3u) ? (nb - 1u) * BS : (nb - 4u) * BS;
#pragma unroll
                for (int r = 0; r < R; r++)
#pragma unroll
                    for (int q = 0; q < NP; q++) base[r][q] -= inc;
            }
        }
    }
}


// ============================================================================ fused find+compare
// the comparer consumes the finder's per-word PAM masks directly.  Each
// CTA grabs ranges of FGRAB word pairs (dynamic), expands the set bits of its strand into
// a shared-memory queue of positions (block scan -> ordered), and runs the table
// comparison on full batches of CT*R queued items; leftovers carry over to the next grab.
// No item list is written or read (4 B/item x 2), and the finder shrinks to its pass 1.
constexpr uint32_t FGRAB = 32;            // word pairs per grab (one per lane of a warp)
constexpr uint32_t FWQ = 256;             // per-warp ring of queued positions (multiple of 32 * R)

// Per-warp queues: each warp grabs its own word-pair ranges (dynamic ticket), expands its
// strand's set bits into its ring (warp scan, ordered), and compares full batches of 32*R
// positions; no CTA-wide barrier after the table load, so warps hide each other's latency.
template <int NP, int R, int TC, bool W64>
__global__ void __launch_bounds__(CT, W64 ? 2 : 3) cof_comparer_fused(const __grid_constant__ TableArgs a) {
    extern __shared__ __align__(16) uint8_t s_raw[];
    constexpr uint32_t BS = NP * 25 * 8;
    constexpr uint32_t BATCH = 32 * R;
    static_assert(FWQ % BATCH == 0 && FWQ >= 2 * BATCH, "ring");
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t s_raw_a = smem_u32(s_raw);
    const uint32_t s_base = (s_raw_a + 127u) & ~127u;   // table at the first 128-byte boundary
    const uint32_t tab_bytes = (s_base - s_raw_a) + ((a.n_blocks * BS + 15u) & ~15u);
    uint32_t* queue = reinterpret_cast<uint32_t*>(s_raw + tab_bytes) + warp * FWQ;
    {
        const uint2* src = a.ptab;
        uint2* dst = reinterpret_cast<uint2*>(s_raw + (s_base - s_raw_a));
        const uint32_t n8 = a.n_blocks * NP * 25;
        for (uint32_t i = tid; i < n8; i += CT) dst[i] = __ldg(src + i);
    }
    __syncthreads();

    // batches start at multiples of BATCH in the ring, so a batch never wraps
    uint32_t head = 0, q_n = 0;          // warp-uniform
    auto process = [&](uint32_t n_items) {   // ring[head, head + n_items), n_items <= BATCH
        const uint32_t* q = queue + head;
        uint32_t base[R][NP], okm[R];
#pragma unroll
        for (int r = 0; r < R; r++) {
            const uint32_t i = (uint32_t)r * 32 + lane;
            okm[r] = i < n_items ? ~0u : 0u;
            item_bases<NP, W64>(a, s_base, i < n_items ? q[i] : 0u, base[r]);
        }
        if (n_items < BATCH) table_blocks<NP, R, true, TC, 32>(a, base, a.n_blocks, 0, q + lane, okm);
        else table_blocks<NP, R, false, TC, 32>(a, base, a.n_blocks, 0, q + lane, okm);
        __syncwarp();                     // the slots may be refilled after this
        head = (head + BATCH) & (FWQ - 1);
        q_n -= n_items;
    };

    // one ticket = grab_rounds consecutive ranges of FGRAB word pairs (fewer atomics on the
    // shared counter when PAM sites are sparse and a range holds few items)
    uint32_t grab = 0, round = a.grab_rounds;
    for (;;) {
        if (round == a.grab_rounds) {
            if (lane == 0) grab = atomicAdd(a.ticket, 1u);
            grab = __shfl_sync(0xffffffffu, grab, 0);
            round = 0;
        }
        const uint64_t wp0 = ((uint64_t)grab * a.grab_rounds + round++) * FGRAB;
        if (wp0 >= a.n_wp) break;
        const uint64_t wp = wp0 + lane;
        uint32_t m0 = 0, m1 = 0;
        if (wp < a.n_wp) {
            const uint4 v = __ldcs(a.masks + wp);
            m0 = a.strand ? v.y : v.x;
            m1 = a.strand ? v.w : v.z;
        }
        const uint32_t c = (uint32_t)(__popc(m0) + __popc(m1));
        uint32_t x = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        const uint32_t total = __shfl_sync(0xffffffffu, x, 31);
        const uint32_t first = x - c;
        const uint32_t pbase = (uint32_t)(wp * 64);
        for (uint32_t done = 0; done < total;) {
            const uint32_t take = min(FWQ - q_n, total - done);
            const uint32_t tail = head + q_n;
            uint32_t rank = first;
#pragma unroll
            for (int w = 0; w < 2; w++) {
                uint32_t mm = w ? m1 : m0;
                while (mm) {
                    const int b = __ffs(mm) - 1;
                    if (rank - done < take) queue[(tail + rank - done) & (FWQ - 1)] = pbase + 32u * w + (uint32_t)b;
                    rank++;
                    mm &= mm - 1;
                }
            }
            __syncwarp();
            q_n += take;
            done += take;
            while (q_n >= BATCH) process(BATCH);
        }
    }
    while (q_n > 0) process(min(q_n, BATCH));
}

// ============================================================================ host side
struct KernelInfo {
    const void* fn;
    int bps;        // resident CTAs per SM at the launch smem size
    uint32_t smem;
};

static int num_sms() {
    static int sms = -1;
    if (sms < 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    }
    return sms;
}

static cof_status occupancy(const void* fn, uint32_t smem, int* bps) {
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_error(e, "comparer smem attribute");
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, fn, CT, smem);
    if (e != cudaSuccess) return cuda_error(e, "comparer occupancy");
    if (*bps < 1) *bps = 1;
    return COF_OK;
}

constexpr int R_POPC = 8;
constexpr int R_TABLE = 2;   // items per thread

// Tuning knobs (defaults chosen from B200 measurements):
//  COF_TABLE_SMEM_KB     shared-memory budget per CTA for resident guide blocks
static bool g_uniform_t_enabled = getenv("COF_TABLE_GENERIC") == nullptr;
static uint32_t table_smem_budget() {
    static uint32_t v = 0;
    if (!v) {
        const char* e = getenv("COF_TABLE_SMEM_KB");
        v = (e ? (uint32_t)atoi(e) : 72u) * 1024u;
        if (v < 4096) v = 4096;
    }
    return v;
}
static int table_r() { return R_TABLE; }

template <int NP, int R, int TC, bool W64>
static cof_status launch_table_r(TableArgs& t, uint64_t n_hint, cudaStream_t stream) {
    constexpr uint32_t NSLOT = W64 ? 9 : 6;
    // guide blocks resident in shared memory per pass (tiles over blocks if they do not fit)
    const uint32_t per_block = NP * 25 * 8;
    uint32_t bpc = t.n_blocks;
    const uint32_t budget = table_smem_budget();
    if (bpc * per_block > budget) bpc = std::max<uint32_t>(1, budget / per_block);
    t.blocks_per_chunk = bpc;
    const uint32_t smem = 128u + ((bpc * per_block + 15u) & ~15u) + (uint32_t)CT * R * NSLOT * 4u;   // table + window slots
    int bps = 0;
    auto fn = cof_comparer_table<NP, R, TC, W64>;
    cof_status st = occupancy((const void*)fn, smem, &bps);
    if (st != COF_OK) return st;
    uint64_t grid = (uint64_t)num_sms() * bps;
    if (n_hint != ON_DEVICE) {
        const uint64_t tiles = (n_hint + (uint64_t)CT * R - 1) / ((uint64_t)CT * R);
        if (tiles == 0) return COF_OK;
        if (grid > tiles) grid = tiles;
    }
    fn<<<(uint32_t)grid, CT, smem, stream>>>(t);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "cof_comparer_table launch");
    count_launches(1);
    return COF_OK;
}

// Uniform-threshold specializations for the common guide shapes (20-nt SpCas9 guides:
// 10 pairs; 23-nt Cas12a guides: 12 pairs) and t <= 7; everything else runs the generic
// per-guide-threshold kernel.
template <int NP, int R, int TC, bool W64>
static cof_status launch_fused_r(TableArgs& t, cudaStream_t stream) {
    const uint32_t smem = 128u + ((t.n_blocks * NP * 25 * 8 + 15u) & ~15u) + (CT / 32) * FWQ * 4;   // table + rings
    int bps = 0;
    auto fn = cof_comparer_fused<NP, R, TC, W64>;
    cof_status st = occupancy((const void*)fn, smem, &bps);
    if (st != COF_OK) return st;
    const uint64_t grabs = (t.n_wp + FGRAB - 1) / FGRAB;
    uint64_t grid = (uint64_t)num_sms() * bps;
    const uint64_t ctas_needed = (grabs + CT / 32 - 1) / (CT / 32);
    if (grid > ctas_needed) grid = ctas_needed ? ctas_needed : 1;
    fn<<<(uint32_t)grid, CT, smem, stream>>>(t);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "cof_comparer_fused launch");
    count_launches(1);
    return COF_OK;
}

template <int NP, int R, int TC, bool W64 = false>
static cof_status launch_any_r(TableArgs& t, bool fused, uint64_t n_hint, cudaStream_t stream) {
    return fused ? launch_fused_r<NP, R, TC, W64>(t, stream) : launch_table_r<NP, R, TC, W64>(t, n_hint, stream);
}

// Two-word windows (compared span > 32): generic thresholds, one item per thread (the NP
// pair addresses and loaded entries of up to 32 pairs per item), NP a multiple of 4.
template <int NP>
static cof_status launch_table_wide(TableArgs& t, uint64_t n_hint, cudaStream_t stream, bool fused) {
    return launch_any_r<NP, 1, -1, true>(t, fused, n_hint, stream);
}

template <int NP>
static cof_status launch_table(TableArgs& t, int uniform_t, uint64_t n_hint, cudaStream_t stream, bool fused = false) {
    if constexpr (NP == 10 || NP == 12) {
        switch (uniform_t) {
            case 0: return launch_any_r<NP, R_TABLE, 0>(t, fused, n_hint, stream);
            case 1: return launch_any_r<NP, R_TABLE, 1>(t, fused, n_hint, stream);
            case 2: return launch_any_r<NP, R_TABLE, 2>(t, fused, n_hint, stream);
            case 3: return launch_any_r<NP, R_TABLE, 3>(t, fused, n_hint, stream);
            case 4: return launch_any_r<NP, R_TABLE, 4>(t, fused, n_hint, stream);
            case 5: return launch_any_r<NP, R_TABLE, 5>(t, fused, n_hint, stream);
            case 6: return launch_any_r<NP, R_TABLE, 6>(t, fused, n_hint, stream);
            case 7: return launch_any_r<NP, R_TABLE, 7>(t, fused, n_hint, stream);
            default: break;
        }
    }
    return launch_any_r<NP, R_TABLE, -1>(t, fused, n_hint, stream);
}

static uint32_t fused_blocks_per_launch(const cof_plan* plan);
static uint32_t fused_grab_rounds(const cof_plan* plan);

// One launch per (strand, range of <= MAX_TABLE_BLOCKS guide blocks); thresholds travel in
// the parameter space; hit counts accumulate on the device.
static cof_status run_table(const cof_plan* plan, uint8_t* pd, const CompareArgs& a, cudaStream_t stream,
                            const uint4* masks = nullptr, uint64_t n_wp = 0, unsigned int* tickets = nullptr) {
    const bool fused = masks != nullptr;
    static thread_local TableArgs T;   // ~4.5 KB parameter block, one per calling thread
    const uint32_t np = plan->pairs[0].n_pairs;
    int ut = g_uniform_t_enabled ? (int)plan->max_mm[0] : -1;   // same threshold for every guide?
    for (uint32_t i = 1; i < plan->n_guides && ut >= 0; i++)
        if (plan->max_mm[i] != plan->max_mm[0]) ut = -1;
    for (uint32_t sd = 0; sd < 2; sd++) {
        if (!fused && a.n[sd] != ON_DEVICE && a.n[sd] >= (1ull << 32))
            return set_error(COF_E_ARG, "cof_compare: %llu items (item lists index < 2^32 positions)",
                             (unsigned long long)a.n[sd]);
        T.lo = a.lo; T.hi = a.hi; T.nm = a.nm;
        T.items = a.items[sd];
        T.n = a.n[sd];
        T.items_cap = a.items_cap;
        T.hits = a.hits; T.cap = a.cap; T.counters = a.counters;
        T.strand = sd;
        T.pairs = plan->pairs[sd];
        T.masks = masks;
        T.n_wp = n_wp;
        T.ticket = tickets ? tickets + sd : nullptr;
        T.grab_rounds = fused_grab_rounds(plan);
        const uint32_t* pm = (const uint32_t*)(plan->image.data() + (sd == 0 ? plan->lay.pmeta_fwd : plan->lay.pmeta_rev));
        const uint32_t batch = fused ? fused_blocks_per_launch(plan) : MAX_TABLE_BLOCKS;
        for (uint32_t bb = 0, li = 0; bb < plan->n_blocks; bb += batch, li++) {
            if (tickets) T.ticket = tickets + sd * ((plan->n_blocks + batch - 1) / batch) + li;
            T.block_base = bb;
            T.n_blocks = std::min<uint32_t>(batch, plan->n_blocks - bb);
            T.ptab = (const uint2*)(pd + (sd == 0 ? plan->lay.ptab_fwd : plan->lay.ptab_rev)) + (size_t)bb * np * 25;
            for (uint32_t k = 0; k < T.n_blocks; k++)
                for (int w = 0; w < 8; w++) T.meta[k][w] = pm[(size_t)(bb + k) * 8 + w];
            cof_status st;
            if (T.pairs.wide) {
                switch (np) {
                    case 4: st = launch_table_wide<4>(T, T.n, stream, fused); break;
                    case 8: st = launch_table_wide<8>(T, T.n, stream, fused); break;
                    case 12: st = launch_table_wide<12>(T, T.n, stream, fused); break;
                    case 16: st = launch_table_wide<16>(T, T.n, stream, fused); break;
                    case 20: st = launch_table_wide<20>(T, T.n, stream, fused); break;
                    case 24: st = launch_table_wide<24>(T, T.n, stream, fused); break;
                    case 28: st = launch_table_wide<28>(T, T.n, stream, fused); break;
                    case 32: st = launch_table_wide<32>(T, T.n, stream, fused); break;
                    default: return set_error(COF_E_STATE, "cof_compare: %u pairs (wide)", np);
                }
                if (st != COF_OK) return st;
                continue;
            }
            switch (np) {
                case 1: st = launch_table<1>(T, ut, T.n, stream, fused); break;
                case 2: st = launch_table<2>(T, ut, T.n, stream, fused); break;
                case 3: st = launch_table<3>(T, ut, T.n, stream, fused); break;
                case 4: st = launch_table<4>(T, ut, T.n, stream, fused); break;
                case 5: st = launch_table<5>(T, ut, T.n, stream, fused); break;
                case 6: st = launch_table<6>(T, ut, T.n, stream, fused); break;
                case 7: st = launch_table<7>(T, ut, T.n, stream, fused); break;
                case 8: st = launch_table<8>(T, ut, T.n, stream, fused); break;
                case 9: st = launch_table<9>(T, ut, T.n, stream, fused); break;
                case 10: st = launch_table<10>(T, ut, T.n, stream, fused); break;
                case 11: st = launch_table<11>(T, ut, T.n, stream, fused); break;
                case 12: st = launch_table<12>(T, ut, T.n, stream, fused); break;
                case 13: st = launch_table<13>(T, ut, T.n, stream, fused); break;
                case 14: st = launch_table<14>(T, ut, T.n, stream, fused); break;
                case 15: st = launch_table<15>(T, ut, T.n, stream, fused); break;
                case 16: st = launch_table<16>(T, ut, T.n, stream, fused); break;
                default: return set_error(COF_E_STATE, "cof_compare: %u pairs", np);
            }
            if (st != COF_OK) return st;
        }
    }
    return COF_OK;
}

static cof_status launch_popc(const CompareArgs& a, uint64_t tiles_hint, cudaStream_t stream) {
    const uint32_t tab = (2 * a.n_groups + 2 * a.n_recs) * 16;
    const bool smem_ok = tab <= 160 * 1024;
    int bps = 0;
    const void* fn = smem_ok ? (const void*)cof_comparer_popc<R_POPC, true> : (const void*)cof_comparer_popc<R_POPC, false>;
    const uint32_t smem = smem_ok ? tab : 0;
    cof_status st = occupancy(fn, smem, &bps);
    if (st != COF_OK) return st;
    uint64_t grid = (uint64_t)num_sms() * bps;
    if (tiles_hint != ON_DEVICE && grid > tiles_hint) grid = tiles_hint ? tiles_hint : 1;
    if (smem_ok) cof_comparer_popc<R_POPC, true><<<(uint32_t)grid, CT, smem, stream>>>(a);
    else cof_comparer_popc<R_POPC, false><<<(uint32_t)grid, CT, 0, stream>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "cof_comparer_popc launch");
    count_launches(1);
    return COF_OK;
}

static int g_impl = -1;   // 0 = popc, 1 = table (default); COF_COMPARER=popc|table overrides

static int comparer_impl() {
    if (g_impl < 0) {
        const char* e = getenv("COF_COMPARER");
        g_impl = (e && e[0] == 'p') ? 0 : 1;
    }
    return g_impl;
}


cof_status find_launch(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                       uint32_t* items_fwd, uint32_t* items_rev, uint64_t items_cap, bool masks_only,
                       cudaStream_t stream);
const uint4* finder_masks(const void* workspace);
uint64_t finder_word_pairs(const cof_plan* plan, const cof_chunk* dev);
bool single_supported(const cof_plan* plan, bool strict);
uint32_t single_launches(const cof_plan* plan);
cof_status run_single(const cof_plan* plan, uint8_t* pd, const cof_chunk* dev, unsigned int* tickets,
                      uint64_t* hits, uint64_t hits_cap, cudaStream_t stream);

// Guide blocks per launch of the fused comparer: its whole launch table is resident in
// shared memory (no re-loads between mask grabs), so a plan with more blocks runs several
// launches per strand, each re-expanding the finder masks (0.25 B per base).
static uint32_t fused_blocks_per_launch(const cof_plan* plan) {
    const uint32_t per_block = plan->pairs[0].n_pairs * 25u * 8u;
    const size_t avail = table_smem_budget() + 16u * 1024u - (CT / 32) * FWQ * 4u - 1024u;
    return std::min<uint32_t>(MAX_TABLE_BLOCKS, (uint32_t)(avail / per_block));
}
// Word-pair ranges per ticket of the fused comparer: ~16 PAM sites per lane and ticket
// (1 range for NRG; more for sparse PAMs such as Cas12a TTTV), COF_GRAB_ROUNDS overrides.
static uint32_t fused_grab_rounds(const cof_plan* plan) {
    static int env = -2;
    if (env == -2) {
        const char* e = getenv("COF_GRAB_ROUNDS");
        env = e ? atoi(e) : -1;
    }
    if (env > 0) return (uint32_t)std::min(env, 64);
    double d = 1.0;   // expected PAM sites per start and strand on a uniform genome
    for (uint32_t k = 0; k < plan->pam[0].n; k++) d *= __builtin_popcount(plan->pam[0].set[k]) / 4.0;
    const double per_range = d * 64.0;   // per lane (64 starts) and strand
    uint32_t r = 1;
    while (r < 16 && per_range * r < 8.0) r *= 2;
    return r;
}

static bool fusable(const cof_plan* plan) {
    const uint32_t bpl = fused_blocks_per_launch(plan);
    return bpl >= 1 && (plan->n_blocks + bpl - 1) / bpl * 2 <= FUSED_MAX_TICKETS;
}

}  // namespace cof

using namespace cof;

extern "C" {

int cof_find_compare_supported(const cof_plan* plan) {
    return plan && comparer_impl() == 1 && fusable(plan) ? 1 : 0;
}

size_t cof_find_compare_workspace_bytes(uint64_t n_bases) {
    return cof_find_workspace_bytes(n_bases) + FUSED_MAX_TICKETS * sizeof(unsigned int);
}

cof_status cof_find_masks(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace, cof_stream s) {
    if (!plan || !plan_dev || !dev || !workspace) return set_error(COF_E_ARG, "cof_find_masks: NULL argument");
    if (!dev->lo || !dev->hi || !dev->nm) return set_error(COF_E_ARG, "cof_find_masks: chunk planes are NULL");
    cudaStream_t stream = (cudaStream_t)s;
    unsigned long long* counters = (unsigned long long*)((uint8_t*)plan_dev + plan->lay.counters);
    cudaError_t e = cudaMemsetAsync(counters, 0, 2 * sizeof(uint64_t), stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_find_masks memset");
    return find_launch(plan, plan_dev, dev, workspace, nullptr, nullptr, 0, true, stream);
}

cof_status cof_compare_masks(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                             uint64_t* hits, uint64_t hits_cap, uint64_t* n_hits, cof_stream s) {
    if (!plan || !plan_dev || !dev || !workspace || (!hits && hits_cap))
        return set_error(COF_E_ARG, "cof_compare_masks: NULL argument");
    if (!dev->lo || !dev->hi || !dev->nm) return set_error(COF_E_ARG, "cof_compare_masks: chunk planes are NULL");
    if (comparer_impl() != 1 || !fusable(plan))
        return set_error(COF_E_ARG, "cof_compare_masks: guide table too large for the fused kernel "
                                    "(use cof_find_pam + cof_compare)");
    cudaStream_t stream = (cudaStream_t)s;
    uint8_t* pd = (uint8_t*)plan_dev;
    unsigned long long* counters = (unsigned long long*)(pd + plan->lay.counters);
    unsigned int* tickets = (unsigned int*)((uint8_t*)workspace + cof_find_workspace_bytes(dev->n_bases));
    cudaError_t e = cudaMemsetAsync(counters + 2, 0, sizeof(uint64_t), stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(tickets, 0, FUSED_MAX_TICKETS * sizeof(unsigned int), stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_compare_masks memset");
    CompareArgs a;
    a.lo = dev->lo; a.hi = dev->hi; a.nm = dev->nm;
    a.items[0] = a.items[1] = nullptr;
    a.n[0] = a.n[1] = 0;
    a.items_cap = 0;
    a.hits = (unsigned long long*)hits;
    a.cap = hits_cap;
    a.counters = counters;
    const uint64_t n_wp = finder_word_pairs(plan, dev);
    if (n_wp) {
        cof_status st = run_table(plan, pd, a, stream, finder_masks(workspace), n_wp, tickets);
        if (st != COF_OK) return st;
    }
    if (n_hits) {
        uint64_t c = 0;
        e = cudaMemcpyAsync(&c, counters + 2, sizeof c, cudaMemcpyDeviceToHost, stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
        if (e != cudaSuccess) return cuda_error(e, "cof_compare_masks count");
        *n_hits = c;
        if (c > hits_cap)
            return set_error(COF_E_CAPACITY, "cof_compare_masks: %llu hits exceed capacity %llu",
                             (unsigned long long)c, (unsigned long long)hits_cap);
    }
    return COF_OK;
}

int cof_single_supported(const cof_plan* plan) {
    return plan && comparer_impl() == 1 && single_supported(plan, true) &&
           single_launches(plan) <= FUSED_MAX_TICKETS ? 1 : 0;
}

cof_status cof_search_single(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                             uint64_t* hits, uint64_t hits_cap, uint64_t* n_hits, cof_stream s) {
    if (!plan || !plan_dev || !dev || !workspace || (!hits && hits_cap))
        return set_error(COF_E_ARG, "cof_search_single: NULL argument");
    if (!dev->lo || !dev->hi || !dev->nm) return set_error(COF_E_ARG, "cof_search_single: chunk planes are NULL");
    if (!single_supported(plan, false) || single_launches(plan) > FUSED_MAX_TICKETS)
        return set_error(COF_E_ARG, "cof_search_single: the plan's compared span exceeds one 31-position window "
                                    "(use cof_find_compare / cof_find_pam + cof_compare)");
    cudaStream_t stream = (cudaStream_t)s;
    uint8_t* pd = (uint8_t*)plan_dev;
    unsigned long long* counters = (unsigned long long*)(pd + plan->lay.counters);
    unsigned int* tickets = (unsigned int*)((uint8_t*)workspace + cof_find_workspace_bytes(dev->n_bases));
    cudaError_t e = cudaMemsetAsync(counters, 0, 3 * sizeof(uint64_t), stream);
    if (e == cudaSuccess) e = cudaMemsetAsync(tickets, 0, FUSED_MAX_TICKETS * sizeof(unsigned int), stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_search_single memset");
    cof_status st = run_single(plan, pd, dev, tickets, hits, hits_cap, stream);
    if (st != COF_OK) return st;
    if (n_hits) {
        uint64_t c = 0;
        e = cudaMemcpyAsync(&c, counters + 2, sizeof c, cudaMemcpyDeviceToHost, stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
        if (e != cudaSuccess) return cuda_error(e, "cof_search_single count");
        *n_hits = c;
        if (c > hits_cap)
            return set_error(COF_E_CAPACITY, "cof_search_single: %llu hits exceed capacity %llu",
                             (unsigned long long)c, (unsigned long long)hits_cap);
    }
    return COF_OK;
}

cof_status cof_find_compare(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                            uint64_t* hits, uint64_t hits_cap, uint64_t* n_hits, cof_stream s) {
    if (plan && cof_single_supported(plan))   // one streaming kernel
        return cof_search_single(plan, plan_dev, dev, workspace, hits, hits_cap, n_hits, s);
    if (plan && !fusable(plan))
        return set_error(COF_E_ARG, "cof_find_compare: guide table too large for the fused kernel "
                                    "(use cof_find_pam + cof_compare)");
    cof_status st = cof_find_masks(plan, plan_dev, dev, workspace, s);
    if (st != COF_OK) return st;
    return cof_compare_masks(plan, plan_dev, dev, workspace, hits, hits_cap, n_hits, s);
}

cof_status cof_compare(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, const uint32_t* items_fwd,
                       uint64_t n_fwd, const uint32_t* items_rev, uint64_t n_rev, uint64_t* hits, uint64_t hits_cap,
                       uint64_t* n_hits, cof_stream s) {
    if (!plan || !plan_dev || !dev || !items_fwd || !items_rev || (!hits && hits_cap))
        return set_error(COF_E_ARG, "cof_compare: NULL argument");
    if (!dev->lo || !dev->hi || !dev->nm) return set_error(COF_E_ARG, "cof_compare: chunk planes are NULL");
    cudaStream_t stream = (cudaStream_t)s;
    uint8_t* pd = (uint8_t*)plan_dev;
    CompareArgs a;
    a.lo = dev->lo; a.hi = dev->hi; a.nm = dev->nm;
    a.items[0] = items_fwd; a.items[1] = items_rev;
    a.n[0] = n_fwd; a.n[1] = n_rev;
    // the item capacity is only known to the caller; counts from the device are trusted up
    // to n_owned (the finder never reports more than it could write into n_owned slots)
    a.items_cap = dev->n_owned;
    if (n_fwd != ON_DEVICE && n_fwd > a.items_cap) a.items_cap = n_fwd;
    if (n_rev != ON_DEVICE && n_rev > a.items_cap) a.items_cap = n_rev;
    a.hits = (unsigned long long*)hits;
    a.cap = hits_cap;
    a.counters = (unsigned long long*)(pd + plan->lay.counters);
    a.groups[0] = (const uint4*)(pd + plan->lay.groups_fwd);
    a.groups[1] = (const uint4*)(pd + plan->lay.groups_rev);
    a.recs[0] = (const uint4*)(pd + plan->lay.recs_fwd);
    a.recs[1] = (const uint4*)(pd + plan->lay.recs_rev);
    a.n_groups = plan->n_groups;
    a.n_recs = plan->n_recs;

    cudaError_t e = cudaMemsetAsync(a.counters + 2, 0, sizeof(uint64_t), stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_compare memset");
    uint64_t tiles_hint = ON_DEVICE;
    if (n_fwd != ON_DEVICE && n_rev != ON_DEVICE) {
        const int R = comparer_impl() == 0 ? R_POPC : table_r();
        const uint64_t per = (uint64_t)CT * R;
        tiles_hint = (n_fwd + per - 1) / per + (n_rev + per - 1) / per;
    }
    if (tiles_hint != 0) {
        cof_status st;
        if (comparer_impl() == 0 && plan->L <= 32) {   // (v1 records are 32-bit windows)
            st = launch_popc(a, tiles_hint, stream);
        } else {
            st = run_table(plan, pd, a, stream);
        }
        if (st != COF_OK) return st;
    }
    if (n_hits) {
        uint64_t c = 0;
        e = cudaMemcpyAsync(&c, a.counters + 2, sizeof c, cudaMemcpyDeviceToHost, stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
        if (e != cudaSuccess) return cuda_error(e, "cof_compare count");
        *n_hits = c;
        if (c > hits_cap)
            return set_error(COF_E_CAPACITY, "cof_compare: %llu hits exceed capacity %llu", (unsigned long long)c,
                             (unsigned long long)hits_cap);
    }
    return COF_OK;
}

// Select the comparer implementation at run time (0 = popc, 1 = table).  Not part of the
// stable ABI (declared here for tests / benchmarks).
cof_status cof_set_comparer(int impl) {
    if (impl < 0 || impl > 1) return set_error(COF_E_ARG, "cof_set_comparer: impl must be 0 or 1");
    g_impl = impl;
    return COF_OK;
}

}  // extern "C"
