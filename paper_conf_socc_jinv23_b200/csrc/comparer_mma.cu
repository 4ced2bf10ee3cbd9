// Comparer v3 "mma" (cof_comparer_mma): the compare kernel (Listing 1) as an
// int8 GEMM on the 5th-generation tensor cores (tcgen05.mma.kind::i8, accumulators in TMEM).
//
// The paper's kernel walks the non-N query positions of one query per work-item and counts
// genome bases outside the query letter's IUPAC set, keeping the site iff
// the count is <= the threshold.  Over ALL items and ALL guides that count
// is a dense contraction: with the three non-constant Hadamard sign vectors
//     u(A) = (+1,+1,+1)  u(C) = (-1,+1,-1)  u(G) = (+1,-1,-1)  u(T) = (-1,-1,+1)
// u(b).u(b') = 4[b == b'] - 1, and for an IUPAC set S with v(S) = sum_{b in S} u(b),
// u(b).v(S) = 4[b in S] - |S|.  So for a site S (guide orientation) and guide g
//     sum_r u(S_r).v(g_r) = 4 #matches - sum_r |g_r|,
// N-correction columns (a genome N has u = 0 but must count as a mismatch: minus the
// number of Ns per position class times |g_r|) and two constant columns carrying
// c_g = -(4 (n_g - t_g) - sum_r |g_r|) make the accumulator D = 4 (t_g - mm): a hit is
// D >= 0 and mm = t_g - D/4.  All values are small integers, so the s32 accumulation is
// exact and the result is bit-identical to the definition (DESIGN.md §5, §2 G2/G7/G8).
//
// One persistent CTA per SM (19 warps, 96 registers: at most 5 warps per SM sub-partition
// so the 16K-register sub-partition files hold them), warp-specialised:
//   warps 0..15  epilogue: every N-tile is drained by all 16 warps, warp w reading TMEM
//                lanes 32*(w%4) (its lane quarter) x the 32 columns of chunk w/4 with one
//                tcgen05.ld; an AND tree of the 32 accumulators (one LOP3 per two values:
//                all negative <=> no hit) and one vote; a rare slow path buffers the hits
//                per warp in shared memory (one global atomic per 256 keys);
//   warps 16..17 producers: two item rows per thread; load the site's three plane windows
//                (items of tile k+2 and plane words of tile k+1 in flight while tile k is
//                encoded), turn '-' items into guide orientation (bit reverse +
//                complement), spread the sign bits into int8 lanes (one IMUL + one IMAD per
//                4 positions) and store the row in the K-major interleaved layout the MMA
//                reads, with its position in a shared ring;
//   warp 18      TMEM allocation and the MMA issuer (whole warp; one elected lane issues):
//                per item tile and guide tile, KS tcgen05.mma of 128 x tn x 32 into one of
//                four 128-column TMEM accumulators.
// Pipelines: A ring (4 stages; full: producers -> MMA, empty: MMA commit + every epilogue
// warp after the tile's last N-tile), accumulator ring (4 stages; full: MMA commit ->
// epilogue, empty: 16 epilogue warps -> MMA).  The B image of the launch's guide batch
// stays resident in shared memory.
//
// Measured on B200 (tools/microbench_mma.cu, profiles/microbench_mma_r1.txt): i8 MMA
// 8192 MAC/clk/SM back to back, TMEM reads ~430 B/clk/SM with 16 warps; but with K = 64
// (two 32-byte K steps) every N-tile is a short MMA group whose accumulator is written,
// read-modified-written and read back (16 TMEM bytes per comparison), and a group of two
// 64-cycle MMAs costs 300-600 cycles between issue and commit.  End to end this kernel
// reaches ~5.2e12 comparisons/s on C5 (~0.45x the ALU table comparer), so it is an
// alternative implementation (COF_COMPARER=mma / cof_set_comparer(2)), parity-tested, not
// the default.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"

namespace cof {

namespace {

// Role timing (build with -DCOF_MMA_PROFILE and run with COF_MMA_PROF=1): cycles each role
// spends waiting on its barriers, printed per launch to stderr.
#ifdef COF_MMA_PROFILE
#define MMA_PROF_T0(w) long long w = clock64()
#define MMA_PROF_ADD(acc, w) acc += clock64() - w
#else
#define MMA_PROF_T0(w) do {} while (0)
#define MMA_PROF_ADD(acc, w) do {} while (0)
#endif

constexpr int MM_BM = 128;          // items per tile (MMA M, TMEM lanes)
constexpr int MM_STAGES = 4;        // A ring depth
constexpr int MM_ACC = 4;           // accumulator stages in TMEM
constexpr uint32_t MM_ACC_COLS = 128;    // TMEM columns per accumulator stage (tn <= 128)
constexpr uint32_t MM_TMEM_COLS = MM_ACC * MM_ACC_COLS;
// 19 warps: at most 5 per SM sub-partition, so 96 registers per thread fit its 16K registers
constexpr int MM_EPI_WARPS = 16;    // warps 0..15: lane quarter w % 4, 32-column chunk w / 4
constexpr int MM_PROD_WARP0 = MM_EPI_WARPS;   // warps 16..17 (two item rows per thread)
constexpr int MM_PROD_WARPS = 2;
constexpr int MM_MMA_WARP = MM_PROD_WARP0 + MM_PROD_WARPS;   // warp 18
constexpr int MM_THREADS = (MM_MMA_WARP + 1) * 32;
constexpr uint32_t MM_WB = 256;     // per-epilogue-warp hit buffer (keys) in shared memory
constexpr uint64_t MM_ON_DEVICE = COF_COUNT_ON_DEVICE;

struct MmaArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    const uint32_t* items[2];
    uint64_t n[2];                 // MM_ON_DEVICE: counters[0..1]
    uint64_t items_cap;
    unsigned long long* hits;
    uint64_t cap;
    unsigned long long* counters;  // [0] n_fwd [1] n_rev [2] n_hits
    const uint4* bimg;             // B image of the batch (nt * tn rows x kpad bytes)
    const uint8_t* thr;            // t_eff per guide (global guide index)
    uint32_t g0, ng, nt, tn;
    uint32_t L, j0, npos, nclass;
    uint32_t cmask[32];
    unsigned long long* prof;      // optional (COF_MMA_PROF): per-CTA role timings, 8 slots
};

// ---------------------------------------------------------------- tcgen05 / mbarrier helpers
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// mbarrier wait with a suspend-time hint: the waiting warp sleeps in hardware until the
// phase completes instead of spinning on try_wait (spinning warps steal issue slots from
// the epilogue warps that do the work).
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity), "r"(0x989680u)
        : "memory");
}

// Shared-memory matrix descriptor, K-major, no swizzle ("interleaved" core matrices of
// 8 rows x 16 bytes): LBO = 128 B between the two K-adjacent core matrices of a 32-byte
// K step, SBO = distance between 8-row groups; version 1 (sm_100) at bit 46.
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)(128u >> 4) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}

// Instruction descriptor of kind::i8: D s32 (bits 4-5 = 2), A/B signed int8 (bits 7-9,
// 10-12 = 1), both K-major, N >> 3 at bit 17, M >> 4 at bit 24.
__host__ __device__ constexpr uint32_t idesc_i8(uint32_t M, uint32_t N) {
    return (2u << 4) | (1u << 7) | (1u << 10) | ((N >> 3) << 17) | ((M >> 4) << 24);
}

__device__ __forceinline__ void mma_i8(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                       uint32_t accumulate) {
    asm volatile(
        "{\n.reg .pred p;\n"
        "setp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n"
        "}\n" ::"r"(tmem_d),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

__device__ __forceinline__ bool elect_one() {
    uint32_t pred = 0;
    asm volatile(
        "{\n.reg .pred P;\n"
        "elect.sync _|P, 0xffffffff;\n"
        "selp.u32 %0, 1, 0, P;\n"
        "}\n"
        : "=r"(pred));
    return pred != 0;
}

__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, int32_t (&v)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// bits 0..3 of x -> bytes 0..3 (0 or 1)
__device__ __forceinline__ uint32_t spread4(uint32_t x) { return ((x & 0xFu) * 0x00204081u) & 0x01010101u; }

// AND of 32 accumulators (LOP3 a&b&c: one op per two values); sign bit set <=> all < 0
__device__ __forceinline__ int32_t and32(const int32_t (&v)[32]) {
    uint32_t t[11];
#pragma unroll
    for (int i = 0; i < 10; i++) COF_LOP3(t[i], (uint32_t)v[3 * i], (uint32_t)v[3 * i + 1], (uint32_t)v[3 * i + 2], 0x80);
    t[10] = (uint32_t)v[30] & (uint32_t)v[31];
    uint32_t u0, u1, u2, u3;
    COF_LOP3(u0, t[0], t[1], t[2], 0x80);
    COF_LOP3(u1, t[3], t[4], t[5], 0x80);
    COF_LOP3(u2, t[6], t[7], t[8], 0x80);
    COF_LOP3(u3, t[9], t[10], u0, 0x80);
    COF_LOP3(u0, u1, u2, u3, 0x80);
    return (int32_t)u0;
}

struct ItemWin {
    uint32_t lo, hi, nm, pos;   // raw 32-base windows at pos
};

template <int PW, int KS>
__global__ void __launch_bounds__(MM_THREADS, 1) cof_comparer_mma(const __grid_constant__ MmaArgs a) {
    constexpr uint32_t KPAD = 32u * KS;             // bytes per A/B row
    constexpr uint32_t SBO = 8u * KPAD;             // bytes between 8-row groups
    constexpr uint32_t A_STAGE = MM_BM * KPAD;      // bytes per A stage
    constexpr int KW = KS * 8;                      // words per row
    static_assert(3 * PW + 1 <= KW, "row layout");

    extern __shared__ __align__(1024) uint8_t smem[];
    const uint32_t b_bytes = a.nt * a.tn * KPAD;
    uint8_t* sB = smem;
    uint8_t* sA = smem + ((b_bytes + 1023u) & ~1023u);
    uint32_t* sPos = reinterpret_cast<uint32_t*>(sA + MM_STAGES * A_STAGE);                          // [stage][128]
    unsigned long long* sHits = reinterpret_cast<unsigned long long*>(sPos + MM_STAGES * MM_BM);      // [16][MM_WB]
    uint8_t* sThr = reinterpret_cast<uint8_t*>(sHits + MM_EPI_WARPS * MM_WB);                        // [ng]
    uint64_t* bars = reinterpret_cast<uint64_t*>(sThr + ((a.ng + 15u) & ~15u));
    uint64_t* a_full = bars;
    uint64_t* a_empty = bars + MM_STAGES;
    uint64_t* acc_full = bars + 2 * MM_STAGES;
    uint64_t* acc_empty = bars + 2 * MM_STAGES + MM_ACC;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * MM_STAGES + 2 * MM_ACC);

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

    // item counts (device counters of the finder, or host counts)
    uint64_t n0 = a.n[0] == MM_ON_DEVICE ? (uint64_t)a.counters[0] : a.n[0];
    uint64_t n1 = a.n[1] == MM_ON_DEVICE ? (uint64_t)a.counters[1] : a.n[1];
    if (n0 > a.items_cap) n0 = a.items_cap;
    if (n1 > a.items_cap) n1 = a.items_cap;
    const uint64_t ntot = n0 + n1;
    const uint64_t n_tiles = (ntot + MM_BM - 1) / MM_BM;

    // B image -> shared memory (resident for the whole launch)
    {
        const uint32_t n16 = b_bytes / 16u;
        uint4* dst = reinterpret_cast<uint4*>(sB);
        for (uint32_t i = tid; i < n16; i += MM_THREADS) dst[i] = __ldg(a.bimg + i);
        for (uint32_t i = tid; i < a.ng; i += MM_THREADS) sThr[i] = __ldg(a.thr + a.g0 + i);
        fence_proxy_async_smem();
    }
    if (tid == 0) {
        for (int s = 0; s < MM_STAGES; s++) {
            mbar_init(&a_full[s], MM_PROD_WARPS);   // one arrival per producer warp
            mbar_init(&a_empty[s], 1 + MM_EPI_WARPS);   // MMA commit + every epilogue warp (positions)
        }
        for (int s = 0; s < MM_ACC; s++) {
            mbar_init(&acc_full[s], 1);             // MMA commit
            mbar_init(&acc_empty[s], MM_EPI_WARPS); // every epilogue warp drains its chunk
        }
        fence_mbar_init();
    }
    if (warp == MM_MMA_WARP) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(MM_TMEM_COLS)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    long long prof_a = 0, prof_b = 0, prof_c = 0;   // role wait cycles (COF_MMA_PROFILE)
#ifdef COF_MMA_PROFILE
    const long long prof_t0 = clock64();
#endif

    if (warp == MM_MMA_WARP) {
        // ======================================================== MMA issuer
        // the whole warp runs the bookkeeping (warp-uniform values stay in uniform
        // registers); one elected lane issues the MMAs and commits.  Descriptors are
        // precomputed: per stage / guide tile / K step only the start-address field moves.
        const uint32_t idesc = idesc_i8(MM_BM, a.tn);
        const uint64_t ad0 = umma_desc(smem_u32(sA), SBO), bd0 = umma_desc(smem_u32(sB), SBO);
        const uint32_t b_tile = ((a.tn / 8u) * SBO) >> 4;     // descriptor units per guide tile
        uint32_t k = 0, c = 0;
        for (uint64_t t = blockIdx.x; t < n_tiles; t += gridDim.x, k++) {
            const uint32_t s = k % MM_STAGES;
            MMA_PROF_T0(w0);
            mbar_wait_parity(&a_full[s], (k / MM_STAGES) & 1u);
            MMA_PROF_ADD(prof_a, w0);
            tc_fence_after();
            const uint64_t ad = ad0 + (uint64_t)(s * (A_STAGE >> 4));
            uint64_t bd = bd0;
            for (uint32_t j = 0; j < a.nt; j++, c++, bd += b_tile) {
                const uint32_t as = c % MM_ACC;
                MMA_PROF_T0(w1);
                mbar_wait_parity(&acc_empty[as], ((c / MM_ACC) & 1u) ^ 1u);
                MMA_PROF_ADD(prof_b, w1);
                tc_fence_after();
                if (elect_one()) {
                    const uint32_t d = tmem_base + as * MM_ACC_COLS;
#pragma unroll
                    for (int ks = 0; ks < KS; ks++) mma_i8(d, ad + 16u * ks, bd + 16u * ks, idesc, ks > 0 ? 1u : 0u);
                    mma_commit(&acc_full[as]);
                }
                __syncwarp();
            }
            if (elect_one()) mma_commit(&a_empty[s]);
            __syncwarp();
        }
        if (k > 0) {   // drain: the last commit has arrived before the CTA may exit
            const uint32_t s = (k - 1) % MM_STAGES;
            mbar_wait_parity(&a_empty[s], ((k - 1) / MM_STAGES) & 1u);
        }
    } else if (warp >= MM_PROD_WARP0) {
        // ======================================================== producers: item rows
        // thread -> rows r0 + 32 * MM_PROD_WARPS * i (i < RPT)
        constexpr int RPT = MM_BM / (32 * MM_PROD_WARPS);
        const uint32_t r0 = (uint32_t)(warp - MM_PROD_WARP0) * 32u + lane;
        const uint32_t L = a.L, j0 = a.j0;
        const uint32_t span_mask = a.npos >= 32 ? 0xFFFFFFFFu : ((1u << a.npos) - 1u);
        // software pipeline over this CTA's tiles: the items of tile k+2 and the raw plane
        // words of tile k+1 are in flight while tile k is encoded
        auto item_of = [&](uint64_t t, uint32_t r, uint32_t& p, uint32_t& strand) {
            const uint64_t idx = t * MM_BM + r;
            p = 0xFFFFFFFFu; strand = 0;
            if (t < n_tiles && idx < ntot) {
                strand = idx >= n0;
                p = __ldg(a.items[strand] + (strand ? idx - n0 : idx));
            }
        };
        auto words_of = [&](uint32_t p, uint32_t (&wd)[6]) {
            if (p != 0xFFFFFFFFu) {
                const uint32_t wi = p >> 5;
                wd[0] = __ldg(a.lo + wi); wd[1] = __ldg(a.lo + wi + 1);
                wd[2] = __ldg(a.hi + wi); wd[3] = __ldg(a.hi + wi + 1);
                wd[4] = __ldg(a.nm + wi); wd[5] = __ldg(a.nm + wi + 1);
            } else {
                wd[0] = wd[1] = wd[2] = wd[3] = 0u; wd[4] = wd[5] = 0xFFFFFFFFu;
            }
        };
        uint32_t k = 0;
        uint64_t t = blockIdx.x;
        uint32_t p0[RPT], st0[RPT], p1[RPT], st1[RPT], wd0[RPT][6];
#pragma unroll
        for (int i = 0; i < RPT; i++) {
            const uint32_t r = r0 + 32u * MM_PROD_WARPS * i;
            item_of(t, r, p0[i], st0[i]);
            item_of(t + gridDim.x, r, p1[i], st1[i]);
            words_of(p0[i], wd0[i]);
        }
        for (; t < n_tiles; t += gridDim.x, k++) {
            uint32_t p2[RPT], st2[RPT], wd1[RPT][6];
#pragma unroll
            for (int i = 0; i < RPT; i++) {
                item_of(t + 2ull * gridDim.x, r0 + 32u * MM_PROD_WARPS * i, p2[i], st2[i]);
                words_of(p1[i], wd1[i]);
            }
            const uint32_t s = k % MM_STAGES;
            MMA_PROF_T0(w2);
            mbar_wait_sleep(&a_empty[s], ((k / MM_STAGES) & 1u) ^ 1u);
            MMA_PROF_ADD(prof_a, w2);
#pragma unroll
            for (int i = 0; i < RPT; i++) {
                const uint32_t row = r0 + 32u * MM_PROD_WARPS * i;
                const uint32_t pp = p0[i];
                // site in guide orientation, compared span at bit 0
                uint32_t slo = __funnelshift_r(wd0[i][0], wd0[i][1], pp & 31);
                uint32_t shi = __funnelshift_r(wd0[i][2], wd0[i][3], pp & 31);
                uint32_t snm = __funnelshift_r(wd0[i][4], wd0[i][5], pp & 31);
                if (st0[i]) {
                    const uint32_t sh = 32u - L;
                    slo = __brev(~slo) >> sh;
                    shi = __brev(~shi) >> sh;
                    snm = __brev(snm) >> sh;
                }
                slo >>= j0; shi >>= j0; snm = (snm >> j0) & span_mask;
                uint32_t w[KW];
                const uint32_t d2 = slo ^ shi;
#pragma unroll
                for (int x = 0; x < PW; x++) {
                    w[x] = spread4(slo >> (4 * x)) * 0xFEu + 0x01010101u;
                    w[PW + x] = spread4(shi >> (4 * x)) * 0xFEu + 0x01010101u;
                    w[2 * PW + x] = spread4(d2 >> (4 * x)) * 0xFEu + 0x01010101u;
                }
                w[3 * PW] = 0x00000101u;
#pragma unroll
                for (int x = 3 * PW + 1; x < KW; x++) w[x] = 0u;
                if (snm) {   // genome Ns in the span: zero their signs, count them per class
#pragma unroll
                    for (int x = 0; x < PW; x++) {
                        const uint32_t z = ~(spread4(snm >> (4 * x)) * 0xFFu);
                        w[x] &= z; w[PW + x] &= z; w[2 * PW + x] &= z;
                    }
#pragma unroll
                    for (int x = 3 * PW; x < KW; x++) {
#pragma unroll
                        for (int b = 0; b < 4; b++) {
                            const int cl = (x - 3 * PW) * 4 + b - 2;
                            if (cl >= 0 && cl < 32 && (uint32_t)cl < a.nclass) {
                                const uint32_t cnt = (uint32_t)__popc(snm & a.cmask[cl]);
                                w[x] |= ((0u - cnt) & 0xFFu) << (8 * b);
                            }
                        }
                    }
                }
                if (pp == 0xFFFFFFFFu) {   // past the last item: zero row (the epilogue skips it)
#pragma unroll
                    for (int x = 0; x < KW; x++) w[x] = 0u;
                }
                sPos[s * MM_BM + row] = pp;
                uint8_t* rowp = sA + s * A_STAGE + (row / 8u) * SBO + (row % 8u) * 16u;
#pragma unroll
                for (int kc = 0; kc < KW / 4; kc++)
                    *reinterpret_cast<uint4*>(rowp + kc * 128) =
                        make_uint4(w[4 * kc], w[4 * kc + 1], w[4 * kc + 2], w[4 * kc + 3]);
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&a_full[s]);
#pragma unroll
            for (int i = 0; i < RPT; i++) {
                p0[i] = p1[i]; st0[i] = st1[i]; p1[i] = p2[i]; st1[i] = st2[i];
#pragma unroll
                for (int x = 0; x < 6; x++) wd0[i][x] = wd1[i][x];
            }
        }
    } else {
        // ======================================================== epilogue
        // every N-tile is drained by all 16 warps: warp w reads TMEM lanes 32 * (w % 4) (its
        // lane quarter) and the 32 columns of chunk w / 4
        const uint32_t q = (uint32_t)(warp & 3), ch = (uint32_t)(warp >> 2);
        const uint32_t row = q * 32u + lane;
        const bool has_chunk = ch * 32u < a.tn;
        unsigned long long* wbuf = sHits + (uint32_t)warp * MM_WB;
        uint32_t wn = 0;                                  // keys in this warp's buffer (warp-uniform)
        auto flush = [&]() {                              // buffer -> hits (one global atomic)
            unsigned long long base = 0;
            if (lane == 0) base = atomicAdd(&a.counters[2], (unsigned long long)wn);
            base = __shfl_sync(0xFFFFFFFFu, base, 0);
            __syncwarp();
            for (uint32_t i = lane; i < wn; i += 32)
                if (base + i < a.cap) a.hits[base + i] = wbuf[i];
            __syncwarp();
            wn = 0;
        };
        uint32_t c = 0, j = 0, k = 0;
        for (uint64_t t = blockIdx.x; t < n_tiles;) {
            const uint32_t s = k % MM_STAGES;
            const uint32_t as = c % MM_ACC;
            const uint64_t idx = t * MM_BM + row;
            const bool rvalid = idx < ntot;
            MMA_PROF_T0(w3);
            mbar_wait_parity(&acc_full[as], (c / MM_ACC) & 1u);
            MMA_PROF_ADD(prof_a, w3);
            tc_fence_after();
            if (has_chunk) {
                int32_t v[32];
                MMA_PROF_T0(w4);
                tmem_ld32(tmem_base + ((q * 32u) << 16) + as * MM_ACC_COLS + ch * 32u, v);
                tmem_wait_ld();
                MMA_PROF_ADD(prof_b, w4);
                // AND of the 32 accumulators: sign bit clear <=> some accumulator >= 0 (a hit)
                const bool has = rvalid && and32(v) >= 0;
                if (__any_sync(0xFFFFFFFFu, has)) {
                    MMA_PROF_T0(w5);
                    // slow path: hit mask, warp prefix, per-warp shared-memory buffer
                    const uint32_t lg0 = j * a.tn + ch * 32u;    // batch-local guide of v[0]
                    uint32_t m = 0;
                    if (has) {
#pragma unroll
                        for (int i = 0; i < 32; i++) m |= (v[i] >= 0 ? 1u : 0u) << i;
                        if (lg0 + 32u > a.ng) m &= lg0 >= a.ng ? 0u : ((1u << (a.ng - lg0)) - 1u);
                    }
                    const uint32_t cnt = (uint32_t)__popc(m);
                    uint32_t incl = cnt;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
                        if (lane >= o) incl += y;
                    }
                    const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
                    if (total) {
                        if (wn + total > MM_WB) flush();
                        const uint32_t strand = idx >= n0 ? 1u : 0u;
                        const uint32_t pos = sPos[s * MM_BM + row];
                        const unsigned long long hk =
                            ((unsigned long long)pos << 32) | ((unsigned long long)strand << 31);
                        if (total <= MM_WB) {
                            uint32_t o = wn + incl - cnt;
#pragma unroll
                            for (int i = 0; i < 32; i++) {
                                if (m >> i & 1u) {
                                    const uint32_t lg = lg0 + (uint32_t)i;
                                    const uint32_t mm = (uint32_t)sThr[lg] - (uint32_t)(v[i] >> 2);
                                    wbuf[o++] = hk | ((unsigned long long)(a.g0 + lg) << 7) | mm;
                                }
                            }
                            wn += total;
                            __syncwarp();
                        } else {   // more hits than the buffer holds: straight to global memory
                            unsigned long long base = 0;
                            if (lane == 31) base = atomicAdd(&a.counters[2], (unsigned long long)total);
                            base = __shfl_sync(0xFFFFFFFFu, base, 31);
                            unsigned long long o = base + incl - cnt;
#pragma unroll
                            for (int i = 0; i < 32; i++) {
                                if (m >> i & 1u) {
                                    const uint32_t lg = lg0 + (uint32_t)i;
                                    const uint32_t mm = (uint32_t)sThr[lg] - (uint32_t)(v[i] >> 2);
                                    if (o < a.cap) a.hits[o] = hk | ((unsigned long long)(a.g0 + lg) << 7) | mm;
                                    o++;
                                }
                            }
                        }
                    }
                    MMA_PROF_ADD(prof_c, w5);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_empty[as]);
            c++;
            if (++j == a.nt) {   // tile done: its positions (stage s) may be overwritten
                if (lane == 0) mbar_arrive(&a_empty[s]);
                j = 0; k++; t += gridDim.x;
            }
        }
        if (wn) flush();
    }

#ifdef COF_MMA_PROFILE
    if (a.prof && lane == 0) {
        const long long tot = clock64() - prof_t0;
        const int role = warp == MM_MMA_WARP ? 0 : warp >= MM_PROD_WARP0 ? 1 : 2;
        atomicAdd(&a.prof[role * 3 + 0], (unsigned long long)tot);
        atomicAdd(&a.prof[role * 3 + 1], (unsigned long long)prof_a);
        atomicAdd(&a.prof[role * 3 + 2], (unsigned long long)prof_b);
        atomicAdd(&a.prof[9 + role], (unsigned long long)prof_c);
    }
#else
    (void)prof_a; (void)prof_b; (void)prof_c;
#endif
    tc_fence_before();
    __syncthreads();
    if (warp == MM_MMA_WARP) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(MM_TMEM_COLS)
                     : "memory");
    }
}

using MmaFn = void (*)(MmaArgs);

template <int PW>
MmaFn pick_ks(uint32_t ks) {
    constexpr int KS0 = (12 * PW + 3 + 31) / 32;
    if ((int)ks == KS0) return cof_comparer_mma<PW, KS0>;
    if ((int)ks == KS0 + 1) return cof_comparer_mma<PW, KS0 + 1>;
    return nullptr;
}

MmaFn pick_kernel(uint32_t pw, uint32_t ks) {
    switch (pw) {
        case 1: return pick_ks<1>(ks);
        case 2: return pick_ks<2>(ks);
        case 3: return pick_ks<3>(ks);
        case 4: return pick_ks<4>(ks);
        case 5: return pick_ks<5>(ks);
        case 6: return pick_ks<6>(ks);
        case 7: return pick_ks<7>(ks);
        case 8: return pick_ks<8>(ks);
        default: return nullptr;
    }
}

int mma_num_sms() {
    static int sms = -1;
    if (sms < 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    }
    return sms;
}

}  // namespace

bool mma_supported(const cof_plan* plan) {
    const MmaPlan& mp = plan->mma;
    return pick_kernel(mp.pw, mp.ks) != nullptr;
}

// One launch per guide batch over both strands' item lists (fwd tiles then rev tiles).
cof_status run_mma(const cof_plan* plan, uint8_t* pd, const uint32_t* lo, const uint32_t* hi, const uint32_t* nm,
                   const uint32_t* items_fwd, uint64_t n_fwd, const uint32_t* items_rev, uint64_t n_rev,
                   uint64_t items_cap, unsigned long long* hits, uint64_t cap, unsigned long long* counters,
                   cudaStream_t stream) {
    const MmaPlan& mp = plan->mma;
    MmaFn fn = pick_kernel(mp.pw, mp.ks);
    if (!fn) return set_error(COF_E_STATE, "mma comparer: no kernel for pw=%u ks=%u", mp.pw, mp.ks);
    MmaArgs A;
    A.lo = lo; A.hi = hi; A.nm = nm;
    A.items[0] = items_fwd; A.items[1] = items_rev;
    A.n[0] = n_fwd; A.n[1] = n_rev;
    A.items_cap = items_cap;
    A.hits = hits; A.cap = cap; A.counters = counters;
    A.thr = pd + plan->lay.mma_thr;
    A.L = plan->L; A.j0 = mp.j0; A.npos = mp.npos; A.nclass = mp.nclass;
    for (int i = 0; i < 32; i++) A.cmask[i] = mp.cmask[i];
#ifdef COF_MMA_PROFILE
    static const bool prof = getenv("COF_MMA_PROF") != nullptr;
#else
    const bool prof = false;
#endif
    A.prof = nullptr;
    if (prof) {
        cudaMalloc(&A.prof, 16 * sizeof(unsigned long long));
        cudaMemsetAsync(A.prof, 0, 16 * sizeof(unsigned long long), stream);
    }
    uint64_t grid = (uint64_t)mma_num_sms();
    if (n_fwd != MM_ON_DEVICE && n_rev != MM_ON_DEVICE) {
        const uint64_t tiles = (n_fwd + n_rev + MM_BM - 1) / MM_BM;
        if (tiles == 0) return COF_OK;
        if (grid > tiles) grid = tiles;
    }
    for (const MmaBatch& b : mp.batches) {
        A.bimg = (const uint4*)(pd + plan->lay.mma_b + b.b_off);
        A.g0 = b.g0; A.ng = b.ng; A.nt = b.nt; A.tn = b.tn;
        const uint32_t b_bytes = b.nt * b.tn * mp.kpad;
        uint32_t smem = ((b_bytes + 1023u) & ~1023u) + MM_STAGES * MM_BM * (mp.kpad + 4u) +
                        MM_EPI_WARPS * MM_WB * 8u + ((b.ng + 15u) & ~15u) + (2 * MM_STAGES + 2 * MM_ACC) * 8u +
                        16u + 1024u;
        smem = std::max<uint32_t>(smem, 120u * 1024u);   // one CTA per SM (it owns the TMEM columns)
        cudaError_t e = cudaFuncSetAttribute((const void*)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return cuda_error(e, "mma comparer smem attribute");
        fn<<<(uint32_t)grid, MM_THREADS, smem, stream>>>(A);
        e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "cof_comparer_mma launch");
        count_launches(1);
    }
    if (prof) {
        unsigned long long h[16];
        cudaMemcpyAsync(h, A.prof, sizeof h, cudaMemcpyDeviceToHost, stream);
        cudaStreamSynchronize(stream);
        const char* names[3] = {"mma", "producer", "epilogue"};
        const char* wa[3] = {"wait a_full", "wait a_empty", "wait acc_full"};
        const char* wb[3] = {"wait acc_empty", "-", "tmem ld+wait"};
        for (int r = 0; r < 3; r++)
            fprintf(stderr, "[mma prof] %-8s total %.3e  %s %.1f%%  %s %.1f%%  slow %.1f%%\n", names[r], (double)h[r * 3],
                    wa[r], 100.0 * h[r * 3 + 1] / (h[r * 3] + 1), wb[r], 100.0 * h[r * 3 + 2] / (h[r * 3] + 1),
                    100.0 * h[9 + r] / (h[r * 3] + 1));
        cudaFree(A.prof);
    }
    return COF_OK;
}

}  // namespace cof
