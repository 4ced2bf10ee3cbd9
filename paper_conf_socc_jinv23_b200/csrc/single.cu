// Single-pass find + compare for sm_100a: ONE streaming kernel tests the
// PAM on both strands and compares every passing site against every guide of the launch,
// so neither item lists (4 B per item, written and re-read) nor PAM masks ever reach HBM.
//
// Paper: the host hands the search kernel's PAM sites to the compare kernel; the
// compare kernel (Listing 1) counts, per site and query, the mismatched bases
// over the query's non-N positions and appends a hit when the count is
// <= the threshold through an atomic counter.
//
// B200 design (DESIGN.md §5 "Single pass"):
//  * persistent CTAs, one per SM, streaming tiles of the lo / hi / nm (/ vs) planes
//    through a 4-stage shared-memory ring filled by the TMA engine (cp.async.bulk +
//    mbarrier); tiles are grabbed dynamically (one global atomic per tile), and the
//    refill of a stage is issued by whichever warp releases it last (a shared-memory
//    counter per stage) -- no producer warp, no blocking on an "empty" barrier;
//  * 16 warps, one plane word (32 window starts) per lane: the lane copies its three
//    words of each plane into registers, releases the stage at once, evaluates the
//    pattern and its reverse complement bit-parallel (the finder's multiplexer test), and
//    appends every passing start to its warp's ring queue together with the start's three
//    32-bit window slices (funnel shifts of the registers: no global window gathers);
//  * full batches of 64 queued sites (2 per lane) are compared against the launch's guide
//    blocks in two steps:
//      filter -- per site, position pair q and 32-guide block, one 32-bit shared-memory
//        lookup indexed by the pair's two genome bases gives "the pair holds >= 1
//        mismatch" for all 32 guides; a carry-save tree counts those bits, and a guide
//        survives iff the count of mismatched pairs is <= its threshold.  Every mismatch
//        lies in some pair, so #mismatched pairs <= #mismatches: a hit always survives
//        (necessary condition), while on a random genome only ~0.3% of (site, guide)
//        comparisons do at t = 6 (about 70x the hit rate);
//      verify -- each survivor's exact count from its record: popc over the compared
//        positions of (window != guide) | N (Listing 1's rows, bit-parallel), or the
//        one-hot IUPAC form for degenerate letters; hits are appended warp-aggregated
//        (one atomic per warp and round).
//    Per comparison that is ~0.5 ALU op + 0.3 shared-memory lookups of the filter plus the
//    rare verifications, against ~1.2 + 0.3 (64-bit lookups) for the exact pair-table sum.
#include <algorithm>
#include <mutex>
#include <type_traits>

#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"
#include "csa_gen.cuh"
#include "filter_circuit.cuh"

namespace cof {

// Kernel geometry.  Two instantiations (measured on B200): few guide blocks
// (<= 8: C1-C4) take two sites per lane per batch -- the per-site work (queueing, table
// addresses) is amortised over more lookups -- and 20 warps; many blocks (C5) take one
// site per lane and 28 warps, which hides the filter's dependency latency better and keeps
// all 32 blocks of a 1000-guide plan in one launch's shared memory.
template <int W, int R, int S, int QB, int GUN, int KBN, int WPLN>
struct SCfg {
    static constexpr int SW = W;                  // warps per CTA (one CTA per SM)
    static constexpr int STHREADS = 32 * W;
    static constexpr int STW = 32 * W;            // plane words per tile (one per lane)
    static constexpr int SLOAD = STW + 4;         // words per plane and stage: tile + halo (16-byte multiple)
    static constexpr int SSTAGES = S;             // TMA ring depth
    static constexpr int SR = R;                  // sites per lane and batch
    static constexpr uint32_t SQ = 32u * R * QB;  // queued sites per warp (16-byte entries): QB batches
    static constexpr uint32_t SBATCH = 32u * R;
    static constexpr int GU = GUN;                // groups of 4 guide blocks per filter step
    static constexpr int KB = KBN;                // batches whose survivors may carry over
    static constexpr int WPL = WPLN;              // plane words per lane and chunk
    static constexpr int CPT = W / WPLN;          // chunks per tile
    static_assert(W % WPLN == 0, "whole chunks per tile");
    static_assert((KB + 1) * 32 * R <= 32 * R * QB, "carried batches leave room to append");
    static constexpr uint32_t SVC = 32u * R * GU <= 32u ? 64u : 32u * R * GU <= 96u ? 128u : 256u;   // survivor ring
    static_assert(SQ % SBATCH == 0 && SQ >= 2 * SBATCH && (SQ & (SQ - 1)) == 0, "ring");
    static constexpr uint32_t SPW = 5u * SVC;     // per-warp words of the survivor ring
    static_assert(SPW % 4 == 0, "16-byte survivor masks");
    static_assert(SVC >= 31 + 32 * SR * GU, "a group of blocks appends at most 32 entries per site row");
};
// (warps, sites per lane, ring stages, queue batches); -DCOF_FEW_W=... etc. override for A/B builds
#ifndef COF_FEW_W
#define COF_FEW_W 24
#endif
#ifndef COF_FEW_R
#define COF_FEW_R 2
#endif
#ifndef COF_FEW_S
#define COF_FEW_S 4
#endif
#ifndef COF_FEW_Q
#define COF_FEW_Q 4
#endif
#ifndef COF_MANY_Q
#define COF_MANY_Q 4
#endif
#ifndef COF_FEW_G
#define COF_FEW_G 1
#endif
#ifndef COF_MANY_G
#define COF_MANY_G 2
#endif
#ifndef COF_FEW_K
#define COF_FEW_K 3
#endif
#ifndef COF_MANY_K
#define COF_MANY_K 3
#endif
#ifndef COF_MANY_W
#define COF_MANY_W 28
#endif
#ifndef COF_MANY_R
#define COF_MANY_R 1
#endif
#ifndef COF_MANY_S
#define COF_MANY_S 2
#endif
#ifndef COF_SPARSE_WPL
#define COF_SPARSE_WPL 4
#endif
#ifndef COF_FEW_WPL
#define COF_FEW_WPL 1
#endif
#ifndef COF_MANY_WPL
#define COF_MANY_WPL 1
#endif
using SCfgFew = SCfg<COF_FEW_W, COF_FEW_R, COF_FEW_S, COF_FEW_Q, COF_FEW_G, COF_FEW_K, COF_FEW_WPL>;
// few blocks and a sparse PAM (Cas12a TTTV): several plane words per lane and chunk, so the
// per-chunk work (tile bookkeeping, the append's scan) is spread over more sites
using SCfgSparse = SCfg<COF_FEW_W, COF_FEW_R, COF_FEW_S, COF_FEW_Q, COF_FEW_G, COF_FEW_K, COF_SPARSE_WPL>;
using SCfgMany = SCfg<COF_MANY_W, COF_MANY_R, COF_MANY_S, COF_MANY_Q, COF_MANY_G, COF_MANY_K, COF_MANY_WPL>;
#ifndef COF_FEW_MAXB
#define COF_FEW_MAXB 8
#endif
constexpr uint32_t SFEW_BLOCKS = COF_FEW_MAXB;   // guide blocks up to which SCfgFew runs
constexpr int SPL = 4;                    // planes per stage: lo, hi, nm, vs
constexpr uint32_t SMAX_BLOCKS = 64;      // guide blocks per launch (shared-memory tables)
constexpr uint32_t S_END = 0xFFFFFFFFu;   // tile id: no more tiles

struct SingleArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    const uint32_t* vs;               // valid-start plane (multi-segment chunks) or nullptr
    uint64_t limit;                   // no window start >= limit is valid
    uint32_t n_tiles;
    uint64_t words;                   // plane words allocated (cof_plane_words(n_bases)): TMA bound
    unsigned int* ticket;             // dynamic tile counter (zeroed per launch)
    unsigned long long* hits;
    uint64_t cap;
    unsigned long long* counters;     // [0] n_fwd, [1] n_rev (PAM sites), [2] n_hits
    const uint32_t* ftab[2];          // filter tables of this launch's blocks, per strand
    const uint4* vrec[2];             // verification records of this launch's guides, per strand
    uint32_t n_blocks;                // guide blocks in this launch
    uint32_t block_base;              // first block of this launch (global guide = (base + b) * 32 + k)
    uint32_t count_items;             // count PAM sites (one launch per search does)
    uint32_t ne;                      // non-N pattern letters per strand
    uint32_t pam_hi;                  // some PAM letter sits at window offset >= 32 (L > 32)
    uint32_t pj[2][32];               // their window offsets
    uint4 psel[2][32];                // their IUPAC sets as splat words {A, C, G, T}
    uint32_t p0[2];                   // first compared window offset per strand
    uint32_t contig;                  // compared positions contiguous from p0 (both strands)
    uint32_t cmp_mask;                // n_cmp low bits: the compared positions of a window at p0
    uint32_t j1[2][16], j2[2][16];    // pair offsets relative to p0 (j2 = 0xFF: single position)
    uint32_t meta[SMAX_BLOCKS][8];    // per block: threshold planes T0..T5, valid guide mask
};

// Membership of 32 bases in an IUPAC set given as splat words (the finder's multiplexer);
// a genome N is in no set (reading G2).
__device__ __forceinline__ uint32_t s_member(uint32_t lo, uint32_t hi, uint32_t nm, uint4 sel) {
    const uint32_t t0 = (hi & sel.z) | (~hi & sel.x);
    const uint32_t t1 = (hi & sel.w) | (~hi & sel.y);
    return ((lo & t1) | (~lo & t0)) & ~nm;
}

template <uint32_t OFF>
__device__ __forceinline__ uint32_t lds32(uint32_t addr) {
    uint32_t x;
    asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(x) : "r"(addr), "n"(OFF));
    return x;
}

// The NP filter lookups of one site in block b: pair q at base[q] + boff + OFF + q * 64.
// boff (the group's block offset) is warp-uniform: the address add can live in the
// uniform datapath instead of NP vector adds per site and group.
template <int NP, uint32_t OFF, int Q = 0>
__device__ __forceinline__ void lds_filter(const uint32_t (&base)[NP], uint32_t boff, uint32_t (&v)[NP]) {
    if constexpr (Q < NP) {
        v[Q] = lds32<OFF + (uint32_t)Q * 64u>(base[Q] + boff);
        lds_filter<NP, OFF, Q + 1>(base, boff, v);
    }
}

// Shared-memory addresses of the NP filter entries of a site (pair q's entry read at
// base[q] + q * 64 + block offset); tbase = the strand's table (64-byte aligned).
template <int NP>
__device__ __forceinline__ void site_bases(const SingleArgs& a, uint32_t tbase, uint32_t sd, uint32_t wl,
                                           uint32_t wh, uint32_t wn, uint32_t (&base)[NP]) {
    if (a.contig) {
        // pair q = window offsets (2q, 2q + 1): its 4-bit entry index lo(b1) | lo(b2) << 1 |
        // hi(b1) << 2 | hi(b2) << 3 is nibble q/2 of Y (even q) or Z (odd q)
        const uint32_t Y = (wl & 0x33333333u) | ((wh & 0x33333333u) << 2);
        const uint32_t Z = ((wl >> 2) & 0x33333333u) | (wh & 0xCCCCCCCCu);
#pragma unroll
        for (int q = 0; q < NP; q++) {
            const uint32_t src = (q & 1) ? Z : Y;
            const int k = q >> 1;
            const uint32_t off = k == 0 ? (src << 2) & 0x3Cu : (src >> (4 * k - 2)) & 0x3Cu;
            base[q] = tbase | off;
        }
        return;
    }
#pragma unroll
    for (int q = 0; q < NP; q++) {
        const uint32_t j1 = a.j1[sd][q], j2 = a.j2[sd][q];
        // (a genome N reads as the A of its planes: the filter tables have no N entries)
        const uint32_t b1 = ((wl >> j1) & 1u) | (((wh >> j1) & 1u) << 1);
        uint32_t b2 = 0;
        if (j2 < 32u) b2 = ((wl >> j2) & 1u) | (((wh >> j2) & 1u) << 1);
        base[q] = tbase + pair_entry(NP, (uint32_t)q, b1, b2) * 4u - (uint32_t)q * 64u;
    }
}

__device__ __forceinline__ unsigned long long s_key(uint32_t pos, uint32_t strand, uint32_t guide, uint32_t mm) {
    return ((unsigned long long)pos << 32) | ((unsigned long long)strand << 31) | ((unsigned long long)guide << 7) |
           (unsigned long long)mm;
}

// NE: non-N PAM letters per strand when known at compile time (2: NRG / NGG, 4: TTTV), so the
// PAM test is unrolled with constant parameter offsets; -1: any count (a loop).
template <int NP, int TC, bool CONCRETE, class CFG, int NE = -1>
__global__ void __launch_bounds__(CFG::STHREADS, 1) cof_single_kernel(const __grid_constant__ SingleArgs a) {
    constexpr int SW = CFG::SW, STHREADS = CFG::STHREADS, STW = CFG::STW, SLOAD = CFG::SLOAD;
    constexpr int SSTAGES = CFG::SSTAGES, SR = CFG::SR;
    constexpr uint32_t SQ = CFG::SQ, SBATCH = CFG::SBATCH, SVC = CFG::SVC;
    constexpr int GU = CFG::GU;
    constexpr int WPL = CFG::WPL, CPT = CFG::CPT;
    extern __shared__ __align__(128) uint8_t smem[];
    // layout: [filter tables: '+' n_blocks x FBW words, 64 B, '-' likewise]
    //         [verification records: '+' n_blocks*32 x VS uint4, 64 B, '-' likewise]
    //         [ring: SSTAGES x SPL x SLOAD words][site queues: SW x SQ x uint4]
    //         [per warp: survivor ring (SVC x 5 words)]
    //         [tile ids, release counters][full mbarriers]
    constexpr uint32_t FBW = NP * 16u;
    constexpr uint32_t VSTR = CONCRETE ? 1u : 2u;     // uint4 per verification record in shared memory
    const uint32_t nb = a.n_blocks;
    uint32_t* s_ftab = reinterpret_cast<uint32_t*>(smem);
    uint4* s_vrec = reinterpret_cast<uint4*>(smem + 2 * nb * FBW * 4 + 64);
    uint32_t* ring = reinterpret_cast<uint32_t*>(reinterpret_cast<uint8_t*>(s_vrec) + 2 * nb * 32 * VSTR * 16 + 64);
    uint4* queues = reinterpret_cast<uint4*>(ring + SSTAGES * SPL * SLOAD);
    uint32_t* survs = reinterpret_cast<uint32_t*>(queues + SW * SQ);    // per warp: SPW words
    uint32_t* s_tile = survs + SW * CFG::SPW;
    uint32_t* s_rel = s_tile + SSTAGES;
    uint32_t* s_next = s_rel + SSTAGES;                              // next chunk to take (ring order)
    uint64_t* full = reinterpret_cast<uint64_t*>(s_tile + 2 * SSTAGES + 2);

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const bool vsp = a.vs != nullptr;
    // grab the next tile and stream it into stage st (or mark the stage as the end)
    auto refill = [&](int st) {
        const uint32_t tile = atomicAdd(a.ticket, 1u);
        if (tile >= a.n_tiles) {
            s_tile[st] = S_END;
            __threadfence_block();        // (the arrive releases it too; racecheck wants the fence)
            mbar_arrive(&full[st]);
            return;
        }
        s_tile[st] = tile;
        const size_t w0 = (size_t)tile * STW;
        // (a tile size that does not divide the planes' 512-word padding: the last tile's
        // copy stops at the allocation; the words past it only feed invalid starts)
        COF_ASSERT(w0 < a.words, "single: tile inside the planes");
        const uint32_t nbytes = (uint32_t)min((uint64_t)SLOAD, a.words - w0) * 4u;
        uint32_t* S = ring + st * SPL * SLOAD;
        fence_proxy_async_smem();
        mbar_arrive_expect_tx(&full[st], (vsp ? 4 : 3) * nbytes);
        bulk_g2s(S + 0 * SLOAD, a.lo + w0, nbytes, &full[st]);
        bulk_g2s(S + 1 * SLOAD, a.hi + w0, nbytes, &full[st]);
        bulk_g2s(S + 2 * SLOAD, a.nm + w0, nbytes, &full[st]);
        if (vsp) bulk_g2s(S + 3 * SLOAD, a.vs + w0, nbytes, &full[st]);
    };
    {   // guide tables -> shared memory (both strands; strand '-' 64 bytes further: other banks)
        const uint32_t nf = nb * FBW;
        for (uint32_t i = tid; i < nf; i += STHREADS) {
            s_ftab[i] = __ldg(a.ftab[0] + i);
            s_ftab[nf + 16 + i] = __ldg(a.ftab[1] + i);
        }
        const uint32_t nv = nb * 32;
        for (uint32_t i = tid; i < nv * VSTR; i += STHREADS) {
            const uint32_t g = i / VSTR, h = i % VSTR;
            s_vrec[i] = __ldg(a.vrec[0] + 2 * g + h);
            s_vrec[nv * VSTR + 4 + i] = __ldg(a.vrec[1] + 2 * g + h);
        }
    }
    if (tid == 0) {
        for (int s = 0; s < SSTAGES; s++) {
            mbar_init(&full[s], 1);
            s_rel[s] = 0;
        }
        *s_next = 0;
        fence_mbar_init();
        for (int s = 0; s < SSTAGES; s++) refill(s);
    }
    __syncthreads();

    uint4* queue = queues + warp * SQ;
    uint32_t* sv_x = survs + warp * CFG::SPW;            // survivor entries: slot | group << 8
    uint4* sv_m = reinterpret_cast<uint4*>(sv_x + SVC);  // and the group's 4 survivor masks (16 B)
    const uint32_t tb0 = smem_u32(s_ftab), tb1 = tb0 + nb * FBW * 4 + 64;
    const uint4* vrec1 = s_vrec + nb * 32 * VSTR + 4;
    uint32_t head = 0, q_n = 0;           // warp-uniform site ring state
    // Survivor entries carry over from one batch to the next, up to KB batches (the last
    // verification round of a batch would otherwise run mostly empty): those batches' queue
    // slots stay reserved (resv) until a batch ends with a full drain.
    uint32_t sv_h = 0, sv_n = 0, resv = 0;
    unsigned long long cnt_f = 0, cnt_r = 0;

    // Verify the survivor entries [sv_h, sv_h + n), n <= 32 (one site and the four 32-guide
    // survivor masks of one group of blocks each) in ONE warp-wide round: lane i takes the
    // lowest survivor of entry i, counts its mismatches exactly from the guide's record and
    // clears it; an entry with survivors left goes back to the tail of the ring (ballot
    // append) for a later round.  No per-bit loop: every round verifies one survivor per
    // active lane; the round's hits are appended with one atomic.  Returns
    // the number of entries re-appended.
    auto flush = [&](uint32_t sv_h, uint32_t n, uint32_t tail) -> uint32_t {
        // branch-free: every lane reads an entry slot of the ring (in bounds; stale for lanes
        // >= n, whose masks are zeroed); the stored masks are the filter's FAIL masks (a set
        // bit = no survivor), so the survivors are their complement
        const bool have = (uint32_t)lane < n;
        const uint32_t e = (sv_h + lane) & (SVC - 1);
        const uint32_t x = sv_x[e];
        const uint4 mv = sv_m[e];
        const uint32_t keep = have ? ~0u : 0u;
        uint32_t m0 = ~mv.x & keep, m1 = ~mv.y & keep, m2 = ~mv.z & keep, m3 = ~mv.w & keep;
        const bool z0 = m0 == 0u, z1 = m1 == 0u, z2 = m2 == 0u;
        const uint32_t sel = !z0 ? m0 : (!z1 ? m1 : (!z2 ? m2 : m3));
        const uint32_t bi = !z0 ? 0u : (!z1 ? 32u : (!z2 ? 64u : 96u));
        const uint32_t low = sel & (0u - sel);
        m0 ^= !z0 ? low : 0u;
        m1 ^= z0 && !z1 ? low : 0u;
        m2 ^= z0 && z1 && !z2 ? low : 0u;
        m3 ^= z0 && z1 && z2 ? low : 0u;
        const bool any = sel != 0u;
        const uint32_t g = any ? (x >> 8) * 128u + bi + (31u - (uint32_t)__clz(low)) : 0u;   // launch-local guide
        COF_ASSERT(g < a.n_blocks * 32u, "single: survivor guide inside the launch");
        const uint4 it = queue[x & (SQ - 1)];
        const uint32_t pos = it.x, sd = it.w >> 31;
        const uint32_t wl = it.y, wh = it.z, wn = it.w & 0x7FFFFFFFu;
        const uint4* rec = (sd ? vrec1 : s_vrec) + g * VSTR;
        const uint4 r0 = rec[0];                                      // {lo, hi, care, t}
        uint32_t mis;
        if constexpr (CONCRETE) {
            mis = ((wl ^ r0.x) | (wh ^ r0.y) | wn) & r0.z;
        } else {
            const uint4 oh = rec[1];                                  // one-hot {A, C, G, T}
            const uint32_t nn = ~wn;
            const uint32_t match = (oh.x & ~wl & ~wh & nn) | (oh.y & wl & ~wh & nn) |
                                   (oh.z & ~wl & wh & nn) | (oh.w & wl & wh & nn);
            mis = r0.z & ~match;
        }
        const uint32_t mm = (uint32_t)__popc(mis);
        const bool hit = any && mm <= r0.w;
        const unsigned hm = __ballot_sync(0xFFFFFFFFu, hit);
        if (hm) {
            const int leader = __ffs(hm) - 1;
            unsigned long long o = 0;
            if (lane == leader) o = atomicAdd(&a.counters[2], (unsigned long long)__popc(hm));
            o = __shfl_sync(0xFFFFFFFFu, o, leader) + (unsigned)__popc(hm & lanemask_lt());
            if (hit && o < a.cap) a.hits[o] = s_key(pos, sd, a.block_base * 32u + g, mm);
        }
        // entries with survivors left -> back to the ring's tail (their slots were just read)
        const bool more = (m0 | m1 | m2 | m3) != 0u;
        const unsigned mb = __ballot_sync(0xFFFFFFFFu, more);
        __syncwarp();
        if (more) {
            const uint32_t e = (tail + (uint32_t)__popc(mb & lanemask_lt())) & (SVC - 1);
            sv_x[e] = x;
            sv_m[e] = make_uint4(~m0, ~m1, ~m2, ~m3);
        }
        return (uint32_t)__popc(mb);
    };

    // per-lane state of the tile being appended: its plane words and the PAM bits not yet queued
    // (WPL consecutive plane words per lane and chunk: lo[q] .. lo[q + 2] hold word q's windows)
    uint32_t lo[WPL + 2], hi[WPL + 2], nm[WPL + 2], pend[2][WPL];
#pragma unroll
    for (int q = 0; q < WPL + 2; q++) lo[q] = hi[q] = nm[q] = 0u;
#pragma unroll
    for (int q = 0; q < WPL; q++) pend[0][q] = pend[1][q] = 0u;
    uint32_t pbase = 0;
    bool tiles_done = false;
    // One loop, one call site each for the batch comparison and the queue append (the
    // kernel's code stays small): compare while a full batch is queued, else append the
    // pending sites of the current tile, else take the next tile.
    for (;;) {
        if (q_n >= SBATCH || (tiles_done && (q_n > 0 || sv_n > 0))) {   // (an empty last batch drains)
            // ---------------- compare a batch: ring[head, head + n_items)
            const uint32_t n_items = min(q_n, SBATCH);
            uint32_t base[SR][NP];
#pragma unroll
            for (int r = 0; r < SR; r++) {
                const uint32_t i = (uint32_t)r * 32 + lane;
                // (a missing site of a partial batch appends no survivor)
                const uint4 e = i < n_items ? queue[(head + i) & (SQ - 1)] : make_uint4(0u, 0u, 0u, 0u);
                const uint32_t sd = e.w >> 31;
                site_bases<NP>(a, sd ? tb1 : tb0, sd, e.y, e.z, e.w & 0x7FFFFFFFu, base[r]);
            }

            // steps of GU groups of 4 blocks (immediate table offsets inside a step); one extra
            // pass (b >= nb) drains the survivor list, so the verification code exists once in
            // the kernel (its size decides the I-cache hit rate)
            for (uint32_t b = 0;; b += 4 * GU) {
                const bool drain = b >= nb;
                if (!drain) {
                    const uint32_t boff = b * FBW * 4;
                    // one group: blocks b + 4G .. b + 4G + 3
                    auto group = [&](auto G) {
                        constexpr uint32_t GO = (uint32_t)decltype(G)::value * 4u * FBW * 4u;
                        const uint32_t bg = b + (uint32_t)decltype(G)::value * 4u;
                        const uint32_t* m = a.meta[bg];     // (read by the generic kernel only)
#pragma unroll
                        for (int r = 0; r < SR; r++) {
                            uint32_t v[NP], p0, p1, p2, p3;
                            lds_filter<NP, GO + 0 * FBW * 4>(base[r], boff, v);
                            p0 = filter_pass<NP, TC>(v, m);
                            lds_filter<NP, GO + 1 * FBW * 4>(base[r], boff, v);
                            p1 = filter_pass<NP, TC>(v, m + 8);
                            lds_filter<NP, GO + 2 * FBW * 4>(base[r], boff, v);
                            p2 = filter_pass<NP, TC>(v, m + 16);
                            lds_filter<NP, GO + 3 * FBW * 4>(base[r], boff, v);
                            p3 = filter_pass<NP, TC>(v, m + 24);
                            // a site with a survivor in this group of 4 blocks -> one survivor
                            // entry (ballot append; guides past the plan never survive; a
                            // missing site of a partial batch appends nothing)
                            const bool has = (p0 | p1 | p2 | p3) != 0u && (uint32_t)r * 32u + lane < n_items;
                            const unsigned hb = __ballot_sync(0xFFFFFFFFu, has);
                            const uint32_t e = (sv_h + sv_n + (uint32_t)__popc(hb & lanemask_lt())) & (SVC - 1);
                            if (has) {
                                sv_x[e] = ((head + (uint32_t)r * 32 + lane) & (SQ - 1)) | ((bg >> 2) << 8);
                                sv_m[e] = make_uint4(~p0, ~p1, ~p2, ~p3);   // fail masks (see flush)
                            }
                            sv_n += (uint32_t)__popc(hb);
                            COF_ASSERT(sv_n <= SVC, "single: survivor ring capacity");
                            COF_ASSERT(bg < SMAX_BLOCKS && bg < nb, "single: guide block index");
                        }
                    };
                    group(std::integral_constant<int, 0>{});
                    if constexpr (GU > 1) {
                        if (b + 4 < nb) group(std::integral_constant<int, 1>{});
                    }
                }
                __syncwarp();
                // (at most 31 + SR x GU x 32 entries are queued: SVC holds them; a round takes 32 and
                // puts back at most 32, and every round verifies one survivor per entry taken)
                // (a batch that keeps its survivors for the next one verifies only full rounds)
                const bool keep = resv < (uint32_t)CFG::KB * SBATCH && n_items == SBATCH && !tiles_done;
                while (sv_n >= 32 || (drain && !keep && sv_n > 0)) {
                    const uint32_t nf = min(sv_n, 32u);
                    COF_ASSERT(nf <= 32 && sv_n <= SVC, "single: verification round size");
                    const uint32_t back = flush(sv_h, nf, sv_h + sv_n);
                    sv_h = (sv_h + nf) & (SVC - 1);
                    sv_n = sv_n - nf + back;
                    COF_ASSERT(sv_n <= SVC && back <= nf, "single: survivors re-appended");
                    __syncwarp();
                }
                if (drain) break;
            }
            __syncwarp();
            head = (head + SBATCH) & (SQ - 1);
            q_n -= n_items;
            // this batch's slots stay reserved while survivors may still reference them; after a
            // full drain nothing is pending
            resv = (sv_n > 0u) ? resv + SBATCH : 0u;
            continue;
        }
        if (tiles_done) break;
        uint32_t anyp = 0u;
#pragma unroll
        for (int q = 0; q < WPL; q++) anyp |= pend[0][q] | pend[1][q];
        if (__any_sync(0xFFFFFFFFu, anyp != 0u)) {
            // ---------------- append pending sites: a warp scan ranks the lanes' sites ('+' before
            // '-' within a lane), and every lane writes the queue entries of its own sites that fit
            // (rank < take), each the site's three 32-base windows funnel-shifted out of the
            // lane's registers at the strand's first compared offset p0 (bit 31 of the N window
            // carries the strand).  The order of entries in the queue is immaterial (hits are
            // sorted afterwards); a site that does not fit stays pending for the next append.
            uint32_t cs[2] = {0u, 0u};
#pragma unroll
            for (int q = 0; q < WPL; q++) {
                cs[0] += (uint32_t)__popc(pend[0][q]);
                cs[1] += (uint32_t)__popc(pend[1][q]);
            }
            const uint32_t c = cs[0] + cs[1];
            uint32_t x = c;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, o);
                if (lane >= o) x += y;
            }
            const uint32_t total = __shfl_sync(0xFFFFFFFFu, x, 31);
            COF_ASSERT(q_n + resv <= SQ, "single: site queue occupancy");
            const uint32_t take = min(SQ - q_n - resv, total);
            const uint32_t first = x - c;
            uint32_t left = min(c, take > first ? take - first : 0u);   // this lane's sites that fit
            const uint32_t pw = pbase + (uint32_t)lane * 32u * WPL;      // first start of this lane's words
            uint32_t slot = head + q_n + first;
#pragma unroll
            for (int sd = 0; sd < 2; sd++) {
                const uint32_t ns = min(left, cs[sd]);
                if (ns) {
                    const uint32_t p0 = a.p0[sd];
                    const uint32_t sbit = sd ? 0x80000000u : 0u;
                    uint32_t L[WPL + 1], H[WPL + 1], N[WPL + 1];   // words shifted to the strand's offset p0
#pragma unroll
                    for (int q = 0; q <= WPL; q++) {
                        L[q] = __funnelshift_r(lo[q], lo[q + 1], p0);
                        H[q] = __funnelshift_r(hi[q], hi[q + 1], p0);
                        N[q] = __funnelshift_r(nm[q], nm[q + 1], p0);
                    }
                    uint32_t todo = ns;
#pragma unroll
                    for (int q = 0; q < WPL; q++) {
                        uint32_t m = pend[sd][q];
                        while (todo && m) {
                            const uint32_t low = m & (0u - m);
                            const uint32_t bit = 31u - (uint32_t)__clz(low);
                            m ^= low;
                            todo--;
                            queue[slot & (SQ - 1)] = make_uint4(pw + 32u * q + bit, __funnelshift_r(L[q], L[q + 1], bit),
                                                                __funnelshift_r(H[q], H[q + 1], bit),
                                                                (__funnelshift_r(N[q], N[q + 1], bit) & 0x7FFFFFFFu) | sbit);
                            slot++;
                        }
                        pend[sd][q] = m;
                    }
                    left -= ns;
                }
            }
            __syncwarp();
            q_n += take;
            COF_ASSERT(q_n + resv <= SQ, "single: site queue capacity");
            continue;
        }
        // ---------------- next chunk of 32 plane words (any warp may take any chunk of the
        // ring's tiles, in order: no fixed word ownership, so a warp that is ahead simply takes
        // more chunks instead of waiting for the slowest warp to release the stage)
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(s_next, 1u);
        c = __shfl_sync(0xFFFFFFFFu, c, 0);
        const uint32_t kk = c / (uint32_t)CPT, chunk = c % (uint32_t)CPT;
        const int st = (int)(kk % SSTAGES);
        mbar_wait_parity_sleep(&full[st], (kk / SSTAGES) & 1u);
        const uint32_t tile = s_tile[st];
        if (tile == S_END) {
            tiles_done = true;
            continue;
        }
        const uint32_t* S = ring + st * SPL * SLOAD;
        const int w = ((int)chunk * 32 + lane) * WPL;
#pragma unroll
        for (int q = 0; q < WPL + 2; q++) {
            lo[q] = S[w + q];
            hi[q] = S[SLOAD + w + q];
            nm[q] = S[2 * SLOAD + w + q];
        }
        uint32_t valid[WPL];
#pragma unroll
        for (int q = 0; q < WPL; q++) valid[q] = vsp ? S[3 * SLOAD + w + q] : ~0u;
        __syncwarp();
        if (lane == 0) {   // the chunk is in registers; the last of the tile's CPT chunks refills the stage
            __threadfence_block();
            if (atomicAdd(&s_rel[st], 1u) == CPT - 1) {
                s_rel[st] = 0;
                __threadfence_block();
                refill(st);
            }
        }
        pbase = (uint32_t)(((uint64_t)tile * STW + chunk * 32u * WPL) * 32u);   // first start of lane 0's words
#pragma unroll
        for (int q = 0; q < WPL; q++) {
            const uint64_t pw = (uint64_t)pbase + ((uint32_t)lane * WPL + q) * 32u;   // first start of word q
            uint32_t v = valid[q];
            if (pw + 32 > a.limit) v &= pw >= a.limit ? 0u : (1u << (uint32_t)(a.limit - pw)) - 1u;
            uint32_t p0m = v, p1m = v;
            const uint32_t ne = NE >= 0 ? (uint32_t)NE : a.ne;
#pragma unroll
            for (uint32_t e = 0; e < (NE >= 0 ? (uint32_t)NE : ne); e++) {
                const uint32_t j0 = a.pj[0][e], j1 = a.pj[1][e];
                if (NE >= 0 || !a.pam_hi) {   // (warp-uniform; the unrolled kernels never see L > 32 PAMs)
                    p0m &= s_member(__funnelshift_r(lo[q], lo[q + 1], j0), __funnelshift_r(hi[q], hi[q + 1], j0),
                                    __funnelshift_r(nm[q], nm[q + 1], j0), a.psel[0][e]);
                    p1m &= s_member(__funnelshift_r(lo[q], lo[q + 1], j1), __funnelshift_r(hi[q], hi[q + 1], j1),
                                    __funnelshift_r(nm[q], nm[q + 1], j1), a.psel[1][e]);
                } else {           // L > 32: a letter at offset >= 32 reads the next word pair
                    const int k0 = (int)(j0 >> 5), k1 = (int)(j1 >> 5);
                    p0m &= s_member(__funnelshift_r(k0 ? lo[q + 1] : lo[q], k0 ? lo[q + 2] : lo[q + 1], j0),
                                    __funnelshift_r(k0 ? hi[q + 1] : hi[q], k0 ? hi[q + 2] : hi[q + 1], j0),
                                    __funnelshift_r(k0 ? nm[q + 1] : nm[q], k0 ? nm[q + 2] : nm[q + 1], j0),
                                    a.psel[0][e]);
                    p1m &= s_member(__funnelshift_r(k1 ? lo[q + 1] : lo[q], k1 ? lo[q + 2] : lo[q + 1], j1),
                                    __funnelshift_r(k1 ? hi[q + 1] : hi[q], k1 ? hi[q + 2] : hi[q + 1], j1),
                                    __funnelshift_r(k1 ? nm[q + 1] : nm[q], k1 ? nm[q + 2] : nm[q + 1], j1),
                                    a.psel[1][e]);
                }
            }
            pend[0][q] = p0m;
            pend[1][q] = p1m;
            if (a.count_items) {
                cnt_f += (unsigned)__popc(p0m);
                cnt_r += (unsigned)__popc(p1m);
            }
        }
    }
    if (a.count_items) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            cnt_f += __shfl_xor_sync(0xFFFFFFFFu, cnt_f, o);
            cnt_r += __shfl_xor_sync(0xFFFFFFFFu, cnt_r, o);
        }
        if (lane == 0) {
            atomicAdd(&a.counters[0], cnt_f);
            atomicAdd(&a.counters[1], cnt_r);
        }
    }
}

// ============================================================================ host side
typedef void (*SingleFn)(SingleArgs);

template <int NP, int TC, bool CONCRETE, int NE = -1>
static SingleFn single_fn_t(int geo) {   // 0: many blocks, 1: few, 2: few + sparse PAM
    return geo == 1 ? cof_single_kernel<NP, TC, CONCRETE, SCfgFew, NE>
         : geo == 2 ? cof_single_kernel<NP, TC, CONCRETE, SCfgSparse, NE> : cof_single_kernel<NP, TC, CONCRETE, SCfgMany, NE>;
}

// The kernel variant a plan runs: uniform-threshold, concrete-letter specialisations for
// the configs' shapes (10 pairs: 20-nt SpCas9 guides; 12: 23-nt Cas12a) with t <= 7,
// else the generic one (per-guide thresholds, one-hot IUPAC verification).
static bool single_uses_concrete(uint32_t np, int tc, bool concrete) {
    return (np == 10 || np == 12) && concrete && tc >= 0 && tc <= 7;
}

template <int NP>
static SingleFn single_fn_np(int tc, bool concrete, int geo, uint32_t ne) {
    if constexpr (NP == 10 || NP == 12) {
        if (concrete) {
            // the configs' shapes (t 4-6, 2 or 4 PAM letters) get the unrolled PAM test
            if (ne == 2 && tc == 4) return single_fn_t<NP, 4, true, 2>(geo);
            if (ne == 2 && tc == 5) return single_fn_t<NP, 5, true, 2>(geo);
            if (ne == 2 && tc == 6) return single_fn_t<NP, 6, true, 2>(geo);
            if (ne == 4 && tc == 4) return single_fn_t<NP, 4, true, 4>(geo);
            if (ne == 4 && tc == 5) return single_fn_t<NP, 5, true, 4>(geo);
            if (ne == 4 && tc == 6) return single_fn_t<NP, 6, true, 4>(geo);
            switch (tc) {
                case 0: return single_fn_t<NP, 0, true>(geo);
                case 1: return single_fn_t<NP, 1, true>(geo);
                case 2: return single_fn_t<NP, 2, true>(geo);
                case 3: return single_fn_t<NP, 3, true>(geo);
                case 4: return single_fn_t<NP, 4, true>(geo);
                case 5: return single_fn_t<NP, 5, true>(geo);
                case 6: return single_fn_t<NP, 6, true>(geo);
                case 7: return single_fn_t<NP, 7, true>(geo);
                default: break;
            }
        }
    }
    return single_fn_t<NP, -1, false>(geo);
}

static SingleFn single_fn(uint32_t np, int tc, bool concrete, int geo, uint32_t ne) {
    switch (np) {
        case 1: return single_fn_np<1>(tc, concrete, geo, ne);
        case 2: return single_fn_np<2>(tc, concrete, geo, ne);
        case 3: return single_fn_np<3>(tc, concrete, geo, ne);
        case 4: return single_fn_np<4>(tc, concrete, geo, ne);
        case 5: return single_fn_np<5>(tc, concrete, geo, ne);
        case 6: return single_fn_np<6>(tc, concrete, geo, ne);
        case 7: return single_fn_np<7>(tc, concrete, geo, ne);
        case 8: return single_fn_np<8>(tc, concrete, geo, ne);
        case 9: return single_fn_np<9>(tc, concrete, geo, ne);
        case 10: return single_fn_np<10>(tc, concrete, geo, ne);
        case 11: return single_fn_np<11>(tc, concrete, geo, ne);
        case 12: return single_fn_np<12>(tc, concrete, geo, ne);
        case 13: return single_fn_np<13>(tc, concrete, geo, ne);
        case 14: return single_fn_np<14>(tc, concrete, geo, ne);
        case 15: return single_fn_np<15>(tc, concrete, geo, ne);
        case 16: return single_fn_np<16>(tc, concrete, geo, ne);
        default: return nullptr;
    }
}

struct SGeom {
    int threads, stw, sload, stages;
    uint32_t sq, svc, sw;
};
template <class C>
static SGeom sgeom() { return {C::STHREADS, C::STW, C::SLOAD, C::SSTAGES, C::SQ, C::SVC, (uint32_t)C::SW}; }
static SGeom single_geom(int geo) { return geo == 1 ? sgeom<SCfgFew>() : geo == 2 ? sgeom<SCfgSparse>() : sgeom<SCfgMany>(); }

static size_t single_smem(const SGeom& g, uint32_t np, uint32_t nb, bool concrete) {
    const size_t fbw = filter_block_words(np);
    // (+ 64 bytes after the '+' filter tables and 64 after the '+' records: bank offsets)
    return 2 * nb * fbw * 4 + 64 + 2 * (size_t)nb * 32 * (concrete ? 16 : 32) + 64 +
           (size_t)g.stages * SPL * g.sload * 4 + (size_t)g.sw * g.sq * 16 + (size_t)g.sw * 5 * g.svc * 4 +
           (2 * g.stages + 2) * 4 + g.stages * 8;
}

static constexpr size_t SMEM_MAX = 227 * 1024;

// Guide blocks per launch: as many as fit the shared-memory budget (a multiple of 4).
static uint32_t single_blocks_per_launch(const SGeom& g, uint32_t np, bool concrete) {
    uint32_t nb = SMAX_BLOCKS;
    while (nb > 4 && single_smem(g, np, nb, concrete) > SMEM_MAX) nb -= 4;
    return nb;
}

// The single-pass kernel handles one-word windows: every compared offset of both strands
// within [p0, p0 + 31) (bit 31 of the queued N-window carries the strand), <= 16 pairs.
static bool single_shape_ok(const cof_plan* plan) {
    if (plan->L > 64) return false;
    for (int s = 0; s < 2; s++) {
        const PairLayout& pl = plan->pairs[s];
        // (windows are taken at the strand's first compared offset p0 from a word pair)
        if (pl.wide || pl.n_pairs > 16 || pl.p0 >= 32) return false;
        const uint64_t uc = plan->union_care[s];
        if (!uc) continue;
        const uint32_t span = 64u - (uint32_t)__builtin_clzll(uc) - pl.p0;
        if (span > 31) return false;
    }
    return plan->pairs[0].n_pairs == plan->pairs[1].n_pairs;
}

// The filter pays when few (site, guide) pairs survive it: thresholds well below the pair
// count (COF_SINGLE=1 forces the single pass whenever the shape allows, 0 disables it).
bool single_supported(const cof_plan* plan, bool strict) {
    static int env = -2;
    if (env == -2) {
        const char* e = getenv("COF_SINGLE");
        env = e ? atoi(e) : -1;
    }
    if (env == 0 || !single_shape_ok(plan)) return false;
    if (env == 1 || !strict) return true;
    const uint32_t np = plan->pairs[0].n_pairs;
    uint32_t tmax = 0;
    for (uint32_t i = 0; i < plan->n_guides; i++) tmax = std::max<uint32_t>(tmax, plan->max_mm[i]);
    return tmax + 3 <= np;
}

struct SinglePlanInfo {
    uint32_t np;
    int ut;            // the uniform threshold, -1 if the guides' thresholds differ
    bool concrete;     // the concrete-letter kernel runs
    int geo;           // 0: SCfgMany, 1: SCfgFew, 2: SCfgSparse
    SGeom geom;
    uint32_t bpl;      // guide blocks per launch
};

static SinglePlanInfo single_info(const cof_plan* plan) {
    SinglePlanInfo I;
    I.np = plan->pairs[0].n_pairs;
    I.ut = (int)plan->max_mm[0];
    for (uint32_t i = 1; i < plan->n_guides && I.ut >= 0; i++)
        if (plan->max_mm[i] != plan->max_mm[0]) I.ut = -1;
    I.concrete = single_uses_concrete(I.np, I.ut, !plan->any_degenerate);
    // the few-blocks geometry when the plan's blocks fit one launch of it; its sparse variant
    // when PAM sites are rarer than 0.03 per start and strand on a uniform genome (Cas12a
    // TTTV: 0.012; NRG 0.125, NGG 0.0625)
    const bool few = plan->n_blocks <= SFEW_BLOCKS &&
                     single_smem(single_geom(1), I.np, (plan->n_blocks + 3) & ~3u, I.concrete) <= SMEM_MAX;
    double d = 1.0;
    for (uint32_t k = 0; k < plan->pam[0].n; k++) d *= __builtin_popcount(plan->pam[0].set[k]) / 4.0;
    static int wpl_env = -2;
    if (wpl_env == -2) {
        const char* e = getenv("COF_SPARSE");   // 0: never the sparse geometry, 1: always (tests)
        wpl_env = e ? atoi(e) : -1;
    }
    const bool sparse = wpl_env == 1 || (wpl_env != 0 && d < 0.03);
    I.geo = few ? (sparse ? 2 : 1) : 0;
    I.geom = single_geom(I.geo);
    I.bpl = single_blocks_per_launch(I.geom, I.np, I.concrete);
    return I;
}

static std::mutex g_single_mu;

cof_status run_single(const cof_plan* plan, uint8_t* pd, const cof_chunk* dev, unsigned int* tickets,
                      uint64_t* hits, uint64_t hits_cap, cudaStream_t stream) {
    const uint64_t L = plan->L;
    if (dev->n_bases >= (1ull << 32)) return set_error(COF_E_ARG, "single pass: n_bases must be < 2^32");
    if (((uintptr_t)dev->lo | (uintptr_t)dev->hi | (uintptr_t)dev->nm | (uintptr_t)dev->vs) & 15)
        return set_error(COF_E_ARG, "single pass: planes must be 16-byte aligned");
    if (dev->n_segs && !dev->vs) return set_error(COF_E_ARG, "single pass: multi-segment chunk without vs plane");
    const SinglePlanInfo I = single_info(plan);
    const SGeom& G = I.geom;
    uint64_t limit = dev->n_bases >= L ? dev->n_bases - L + 1 : 0;
    if (!dev->n_segs && limit > dev->n_owned) limit = dev->n_owned;
    const uint32_t n_tiles = (uint32_t)((limit + (uint64_t)G.stw * 32 - 1) / ((uint64_t)G.stw * 32));
    // (the unrolled-PAM kernels assume every PAM letter within the first 32 window offsets)
    bool pam_hi = false;
    for (int s = 0; s < 2; s++)
        for (uint32_t k = 0; k < plan->pam[s].n; k++) pam_hi |= plan->pam[s].j[k] >= 32;
    SingleFn fn = single_fn(I.np, I.ut, I.concrete, I.geo, pam_hi ? 0u : plan->pam[0].n);
    if (!fn) return set_error(COF_E_STATE, "single pass: %u pairs", I.np);
    int dev_id = 0;
    cudaGetDevice(&dev_id);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev_id);
    static thread_local SingleArgs A;
    A.lo = dev->lo; A.hi = dev->hi; A.nm = dev->nm;
    A.vs = dev->n_segs ? dev->vs : nullptr;
    A.limit = limit;
    A.n_tiles = n_tiles;
    A.words = cof_plane_words(dev->n_bases);
    A.hits = (unsigned long long*)hits;
    A.cap = hits_cap;
    A.counters = (unsigned long long*)(pd + plan->lay.counters);
    A.ne = plan->pam[0].n;
    A.pam_hi = 0;
    for (int s = 0; s < 2; s++)
        for (uint32_t k = 0; k < plan->pam[s].n; k++) A.pam_hi |= plan->pam[s].j[k] >= 32 ? 1u : 0u;
    if (plan->pam[1].n != A.ne || A.ne > 32) return set_error(COF_E_STATE, "single pass: PAM letter counts");
    for (int s = 0; s < 2; s++) {
        for (uint32_t k = 0; k < A.ne; k++) {
            const uint32_t set = plan->pam[s].set[k];
            A.pj[s][k] = plan->pam[s].j[k];
            A.psel[s][k] = make_uint4(0u - (set & 1u), 0u - ((set >> 1) & 1u), 0u - ((set >> 2) & 1u),
                                      0u - ((set >> 3) & 1u));
        }
        const PairLayout& pl = plan->pairs[s];
        A.p0[s] = pl.p0;
        for (uint32_t q = 0; q < 16; q++) {
            A.j1[s][q] = q < pl.n_pairs ? pl.j1[q] - pl.p0 : 0u;
            A.j2[s][q] = q < pl.n_pairs && pl.j2[q] < 0xFE ? pl.j2[q] - pl.p0 : 0xFFu;
        }
    }
    A.contig = plan->pairs[0].contig && plan->pairs[1].contig && plan->pairs[0].n_cmp == plan->pairs[1].n_cmp;
    A.cmp_mask = plan->pairs[0].n_cmp >= 32 ? ~0u : ((1u << plan->pairs[0].n_cmp) - 1u);
    const uint32_t fbw = filter_block_words(I.np);
    const uint32_t* pm = (const uint32_t*)(plan->image.data() + plan->lay.pmeta_fwd);
    {
        std::lock_guard<std::mutex> lk(g_single_mu);   // (per device state; cheap, set every call)
        cudaError_t e = cudaFuncSetAttribute((const void*)fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)single_smem(G, I.np, I.bpl, I.concrete));
        if (e != cudaSuccess) return cuda_error(e, "single pass smem attribute");
    }
    uint32_t li = 0;
    for (uint32_t bb = 0; bb < plan->n_blocks; bb += I.bpl, li++) {
        const uint32_t nbl = std::min(I.bpl, plan->n_blocks - bb);
        // whole groups of 4 blocks: padding blocks (zero tables in the plan image) have no valid guide
        const uint32_t nb4 = (nbl + 3) & ~3u;
        A.n_blocks = nb4;
        A.block_base = bb;
        A.count_items = li == 0;
        A.ticket = tickets + li;
        A.ftab[0] = (const uint32_t*)(pd + plan->lay.ftab_fwd) + (size_t)bb * fbw;
        A.ftab[1] = (const uint32_t*)(pd + plan->lay.ftab_rev) + (size_t)bb * fbw;
        A.vrec[0] = (const uint4*)(pd + plan->lay.vrec_fwd) + (size_t)bb * 64;
        A.vrec[1] = (const uint4*)(pd + plan->lay.vrec_rev) + (size_t)bb * 64;
        for (uint32_t k = 0; k < SMAX_BLOCKS; k++)
            for (int w = 0; w < 8; w++) A.meta[k][w] = k < nbl ? pm[(size_t)(bb + k) * 8 + w] : 0u;
        if (n_tiles == 0) continue;
        uint32_t grid = (uint32_t)sms;
        if (grid > n_tiles) grid = n_tiles;
        fn<<<grid, G.threads, single_smem(G, I.np, nb4, I.concrete), stream>>>(A);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "cof_single_kernel launch");
        count_launches(1);
    }
    return COF_OK;
}

uint32_t single_launches(const cof_plan* plan) {
    const SinglePlanInfo I = single_info(plan);
    return (plan->n_blocks + I.bpl - 1) / I.bpl;
}

}  // namespace cof
