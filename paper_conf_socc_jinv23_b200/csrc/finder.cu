// Finder ("search" kernel, M5 + M6) for sm_100a.
//
// Paper: the search kernel selects "specific sites that include a protospacer-adjacent
// motif (PAM)" by a "parallel search over the sites in a chunk"; its signature is
// in Table VI, its body is not printed.  The paper compacts candidate
// loci with an atomic counter (Table V; "the order of updates is not
// deterministic").
//
// B200 design: persistent CTAs stream 256-word tiles of the three
// bit-planes through a 4-stage shared-memory ring filled by the TMA engine
// (cp.async.bulk + mbarrier).  One thread owns one plane word = 32 window starts and
// tests the pattern and its reverse complement bit-parallel: per non-N pattern letter, a
// funnel shift of each plane and a 3-LOP3 multiplexer select membership in the letter's
// IUPAC set, AND-ed over letters.  Passing starts are compacted in order: each CTA owns
// a contiguous tile range, counts it (pass 1), exchanges its total with all CTAs once
// (grid barrier), then walks its pass-1 masks again (pass 2: one warp per tile, warp
// scans of the masks' popcounts, one exchange of tile totals per 8 tiles, ordered direct
// stores).  Algorithmic bytes per base: 3/8 read + 4 x items written (pass 2 re-reads the
// 1/4 B/base of masks, largely from L2).
#include <mutex>

#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"

namespace cof {

constexpr int FT = 256;          // threads per CTA
constexpr int FWPT = 2;          // consecutive plane words (x 32 window starts) per thread
constexpr int FW = FT * FWPT;    // words per tile (16384 window starts)
constexpr int FSTAGES = 4;       // TMA ring depth
constexpr int FLOAD = FW + 4;    // words per plane per stage: tile + halo, 16-byte multiple
constexpr uint32_t FMAX_CTAS = 4096;                      // grid cap (co-residency)
constexpr size_t FWS_BARRIER = 2 * FMAX_CTAS * sizeof(uint64_t);
constexpr size_t FWS_MASKS = FWS_BARRIER + 256;
constexpr int FPL = 4;           // planes per stage: lo, hi, nm, vs (valid starts; multi-segment chunks)
constexpr int FSTAGE_ITEMS = 8192;   // pass 2 (dense): items staged per round, in the idle TMA ring
static_assert(FSTAGE_ITEMS <= FSTAGES * FPL * FLOAD, "pass-2 staging fits the TMA ring");
constexpr uint32_t FSMEM = FSTAGES * FPL * FLOAD * 4 + FSTAGES * 8;

struct FinderArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    const uint32_t* vs;          // valid-start plane or nullptr (then starts [0, limit) are valid)
    uint64_t limit;              // no start >= limit is valid
    uint32_t* out[2];            // '+' / '-' item lists
    uint64_t cap;
    uint64_t* status;            // workspace: per CTA (fwd, rev) totals
    uint32_t* masks;             // workspace: per plane word {fwd, rev} PAM masks (pass 1 -> pass 2)
    unsigned int* barrier;       // workspace: grid barrier counter (zeroed)
    unsigned long long* counters;  // plan_dev counters: [0] n_fwd, [1] n_rev
    uint32_t n_tiles;
    uint32_t stage;              // pass 2 stages items in shared memory (dense PAM sites)
    uint32_t ne;                 // non-N pattern letters per strand (same for both)
    uint32_t pj[2][COF_MAX_L];   // window offset of entry e
    uint4 psel[2][COF_MAX_L];    // entry e's IUPAC set as splat words {A, C, G, T} (0 / ~0)
};

// Membership of each of 32 bases (bit-parallel) in the IUPAC set `set` (A=1 C=2 G=4 T=8):
// a multiplexer on the 2-bit code selects the set bit; N (nm=1) is in no set (G2).
__device__ __forceinline__ uint32_t member(uint32_t lo, uint32_t hi, uint32_t nm, uint4 sel) {
    const uint32_t t0 = (hi & sel.z) | (~hi & sel.x);      // lo = 0: A or G
    const uint32_t t1 = (hi & sel.w) | (~hi & sel.y);      // lo = 1: C or T
    const uint32_t r = (lo & t1) | (~lo & t0);
    return r & ~nm;
}

// PAM masks of the 32 window starts of one plane word, both strands.  NE > 0: entry count
// known at compile time (fully unrolled); NE < 0: generic loop.  WIDE: letters at window
// offsets >= 32 (L > 32) select the plane word pair (w+1, w+2) instead of (w, w+1).
template <int NE, bool WIDE>
__device__ __forceinline__ void pam_masks(const FinderArgs& a, uint32_t valid, const uint32_t* lo,
                                          const uint32_t* hi, const uint32_t* nm, uint32_t (&m)[2]) {
#pragma unroll
    for (int st = 0; st < 2; st++) {
        uint32_t acc = valid;
        const uint32_t n = NE >= 0 ? (uint32_t)NE : a.ne;
#pragma unroll
        for (uint32_t e = 0; e < (NE >= 0 ? (uint32_t)NE : n); e++) {
            const uint32_t j = a.pj[st][e];   // funnel shifts use j & 31
            if (WIDE && (j & 32u)) {
                acc &= member(__funnelshift_r(lo[1], lo[2], j), __funnelshift_r(hi[1], hi[2], j),
                              __funnelshift_r(nm[1], nm[2], j), a.psel[st][e]);
            } else {
                acc &= member(__funnelshift_r(lo[0], lo[1], j), __funnelshift_r(hi[0], hi[1], j),
                              __funnelshift_r(nm[0], nm[1], j), a.psel[st][e]);
            }
        }
        m[st] = acc;
    }
}

// Two passes over a contiguous tile range per CTA with one grid-wide exchange in between:
//  pass 1 counts the passing starts of the CTA's range (no writes), publishes the CTA
//  total and waits at a grid barrier (all CTAs are co-resident: the grid is sized from the
//  occupancy calculator and launched cooperatively); every CTA then sums the totals of the CTAs before it (its global
//  offset) and pass 2 re-streams its range (mostly from L2) and writes the items in order.
// One exchange per CTA replaces a decoupled look-back per tile, whose depth (all
// concurrently running tiles) made it latency-bound.
template <int NE, bool VS, bool MASKS_ONLY, bool WIDE>
__global__ void __launch_bounds__(FT) cof_finder_kernel(const __grid_constant__ FinderArgs a) {
    extern __shared__ __align__(128) uint8_t smem[];
    uint32_t* stage = reinterpret_cast<uint32_t*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + FSTAGES * FPL * FLOAD * 4);
    __shared__ uint32_t s_warp[FT / 32];
    __shared__ uint32_t s_tile_tot;
    __shared__ unsigned long long s_red[FT / 32][2];
    __shared__ unsigned long long s_base[2];

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t per = (a.n_tiles + gridDim.x - 1) / gridDim.x;
    const uint32_t t_begin = min(a.n_tiles, blockIdx.x * per);
    const uint32_t t_end = min(a.n_tiles, t_begin + per);
    const uint32_t n_mine = t_end - t_begin;

    if (tid == 0) {
        for (int s = 0; s < FSTAGES; s++) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();

    auto issue = [&](uint32_t tile, int s) {
        const size_t w0 = (size_t)tile * FW;
        mbar_arrive_expect_tx(&bars[s], (VS ? 4 : 3) * FLOAD * 4);
        bulk_g2s(stage + (s * FPL + 0) * FLOAD, a.lo + w0, FLOAD * 4, &bars[s]);
        bulk_g2s(stage + (s * FPL + 1) * FLOAD, a.hi + w0, FLOAD * 4, &bars[s]);
        bulk_g2s(stage + (s * FPL + 2) * FLOAD, a.nm + w0, FLOAD * 4, &bars[s]);
        if (VS) bulk_g2s(stage + (s * FPL + 3) * FLOAD, a.vs + w0, FLOAD * 4, &bars[s]);
    };

    // ---------------- pass 1: stream the planes (TMA ring), PAM masks -> workspace, counts
    unsigned long long cnt_f = 0, cnt_r = 0;
    if (tid == 0)
        for (int s = 0; s < FSTAGES && (uint32_t)s < n_mine; s++) issue(t_begin + s, s);
    for (uint32_t k = 0; k < n_mine; k++) {
        const uint32_t tile = t_begin + k;
        const int s = (int)(k % FSTAGES);
        mbar_wait_parity(&bars[s], (k / FSTAGES) & 1u);
        const uint32_t* Slo = stage + (s * FPL + 0) * FLOAD + FWPT * tid;
        const uint32_t* Shi = stage + (s * FPL + 1) * FLOAD + FWPT * tid;
        const uint32_t* Snm = stage + (s * FPL + 2) * FLOAD + FWPT * tid;
        const uint32_t* Svs = stage + (s * FPL + 3) * FLOAD + FWPT * tid;
        constexpr int NWD = FWPT + (WIDE ? 2 : 1);   // plane words a thread's windows touch
        uint32_t lo[FWPT + 2], hi[FWPT + 2], nm[FWPT + 2], vsw[FWPT];
#pragma unroll
        for (int w = 0; w < NWD; w++) { lo[w] = Slo[w]; hi[w] = Shi[w]; nm[w] = Snm[w]; }
#pragma unroll
        for (int w = 0; w < FWPT; w++) vsw[w] = VS ? Svs[w] : ~0u;
        __syncthreads();   // every thread has read stage s: refill it
        if (tid == 0 && k + FSTAGES < n_mine) {
            fence_proxy_async_smem();
            issue(tile + FSTAGES, s);
        }
        const uint64_t p0 = ((uint64_t)tile * FW + FWPT * tid) * 32;
        uint32_t mk[2 * FWPT];
#pragma unroll
        for (int w = 0; w < FWPT; w++) {
            const uint64_t pw = p0 + 32u * w;
            uint32_t valid = vsw[w];
            if (pw + 32 > a.limit) valid &= pw >= a.limit ? 0u : (1u << (uint32_t)(a.limit - pw)) - 1u;
            uint32_t mw[2];
            pam_masks<NE, WIDE>(a, valid, lo + w, hi + w, nm + w, mw);
            mk[2 * w] = mw[0];
            mk[2 * w + 1] = mw[1];
            cnt_f += (unsigned)__popc(mw[0]);
            cnt_r += (unsigned)__popc(mw[1]);
        }
        // masks of this thread's FWPT words: {fwd0, rev0, fwd1, rev1} (one 16-byte store)
        reinterpret_cast<uint4*>(a.masks)[(size_t)tile * FT + tid] = make_uint4(mk[0], mk[1], mk[2], mk[3]);
    }

    // ---------------- grid exchange: CTA totals -> this CTA's global offsets
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        cnt_f += __shfl_xor_sync(0xffffffffu, cnt_f, o);
        cnt_r += __shfl_xor_sync(0xffffffffu, cnt_r, o);
    }
    if (lane == 0) { s_red[warp][0] = cnt_f; s_red[warp][1] = cnt_r; }
    __syncthreads();
    if (MASKS_ONLY) {   // fused find+compare: the masks are the output; counts for reporting only
        if (tid == 0) {
            unsigned long long f = 0, r = 0;
            for (int w = 0; w < FT / 32; w++) { f += s_red[w][0]; r += s_red[w][1]; }
            atomicAdd(&a.counters[0], f);
            atomicAdd(&a.counters[1], r);
        }
        return;
    }
    if (tid == 0) {
        unsigned long long f = 0, r = 0;
        for (int w = 0; w < FT / 32; w++) { f += s_red[w][0]; r += s_red[w][1]; }
        st_relaxed_gpu(&a.status[2 * blockIdx.x], f);
        st_relaxed_gpu(&a.status[2 * blockIdx.x + 1], r);
        __threadfence();
        atomicAdd(a.barrier, 1u);
        while (ld_acquire_gpu_u32(a.barrier) < gridDim.x) __nanosleep(64);
    }
    __syncthreads();
    {
        unsigned long long f = 0, r = 0;
        for (uint32_t c = tid; c < blockIdx.x; c += FT) {
            f += ld_relaxed_gpu(&a.status[2 * c]);
            r += ld_relaxed_gpu(&a.status[2 * c + 1]);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            f += __shfl_xor_sync(0xffffffffu, f, o);
            r += __shfl_xor_sync(0xffffffffu, r, o);
        }
        __syncthreads();
        if (lane == 0) { s_red[warp][0] = f; s_red[warp][1] = r; }
        __syncthreads();
        if (tid == 0) {
            unsigned long long bf = 0, br = 0;
            for (int w = 0; w < FT / 32; w++) { bf += s_red[w][0]; br += s_red[w][1]; }
            s_base[0] = bf;
            s_base[1] = br;
            if (blockIdx.x == gridDim.x - 1) {     // last CTA knows the chunk totals
                a.counters[0] = bf + ld_relaxed_gpu(&a.status[2 * blockIdx.x]);
                a.counters[1] = br + ld_relaxed_gpu(&a.status[2 * blockIdx.x + 1]);
            }
        }
        __syncthreads();
    }

    // ---------------- pass 2: masks (workspace, mostly L2) -> ordered item lists
    if (a.stage) {
        // Dense PAM sites: CTA per tile -- thread t scans its 2 words, one CTA scan per
        // tile, items staged in shared memory (the TMA ring, idle after pass 1) and written
        // out coalesced.
        uint32_t* items = stage;
        unsigned long long run_f = 0, run_r = 0;
        const uint4* mptr = reinterpret_cast<const uint4*>(a.masks);
        uint4 mnext = n_mine ? __ldcg(mptr + (size_t)t_begin * FT + tid) : make_uint4(0, 0, 0, 0);
        for (uint32_t k = 0; k < n_mine; k++) {
            const uint32_t tile = t_begin + k;
            const uint4 mv = mnext;
            if (k + 1 < n_mine) mnext = __ldcg(mptr + (size_t)(tile + 1) * FT + tid);
            const uint32_t m[2][FWPT] = {{mv.x, mv.z}, {mv.y, mv.w}};
            const uint32_t cf = (uint32_t)(__popc(mv.x) + __popc(mv.z));
            const uint32_t cr = (uint32_t)(__popc(mv.y) + __popc(mv.w));
            const uint64_t p0 = ((uint64_t)tile * FW + FWPT * tid) * 32;

            // CTA exclusive scan of packed counts (fwd bits 0..15, rev 16..31)
            const uint32_t cnt = cf | (cr << 16);
            uint32_t x = cnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                if (lane >= o) x += y;
            }
            if (lane == 31) s_warp[warp] = x;
            __syncthreads();
            if (warp == 0) {
                uint32_t wv = lane < FT / 32 ? s_warp[lane] : 0u;
                uint32_t wi = wv;
#pragma unroll
                for (int o = 1; o < FT / 32; o <<= 1) {
                    uint32_t y = __shfl_up_sync(0xffffffffu, wi, o);
                    if (lane >= o) wi += y;
                }
                if (lane < FT / 32) s_warp[lane] = wi - wv;
                if (lane == FT / 32 - 1) s_tile_tot = wi;
            }
            __syncthreads();
            const uint32_t local = s_warp[warp] + x - cnt;
            const uint32_t tot = s_tile_tot;
            const uint32_t pbase = (uint32_t)p0;
#pragma unroll
            for (int st = 0; st < 2; st++) {
                const uint32_t total = st == 0 ? (tot & 0xFFFFu) : (tot >> 16);
                const uint32_t first = st == 0 ? (local & 0xFFFFu) : (local >> 16);
                const unsigned long long base = s_base[st] + (st == 0 ? run_f : run_r);
                uint32_t* out = a.out[st];
                // staged in rounds of FSTAGE_ITEMS (one round unless the pattern is very permissive)
                for (uint32_t r0 = 0; r0 < total; r0 += FSTAGE_ITEMS) {
                    if (total <= FSTAGE_ITEMS) {
                        uint32_t off = first;
#pragma unroll
                        for (int w = 0; w < FWPT; w++) {
                            uint32_t mm = m[st][w];
                            while (mm) {
                                const int b = 31 - __clz(mm & (0u - mm));   // (one FLO; __ffs is BREV + FLO)
                                items[off++] = pbase + 32u * w + (uint32_t)b;
                                mm &= mm - 1;
                            }
                        }
                    } else {
                        uint32_t rank = first;
#pragma unroll
                        for (int w = 0; w < FWPT; w++) {
                            uint32_t mm = m[st][w];
                            while (mm) {
                                const int b = 31 - __clz(mm & (0u - mm));   // (one FLO; __ffs is BREV + FLO)
                                if (rank >= r0 && rank < r0 + FSTAGE_ITEMS) items[rank - r0] = pbase + 32u * w + (uint32_t)b;
                                rank++;
                                mm &= mm - 1;
                            }
                        }
                    }
                    __syncthreads();
                    uint32_t n_round = min(total - r0, (uint32_t)FSTAGE_ITEMS);
                    const unsigned long long o0 = base + r0;
                    if (o0 >= a.cap) n_round = 0;
                    else if (a.cap - o0 < n_round) n_round = (uint32_t)(a.cap - o0);
                    uint32_t* __restrict__ dst = out + o0;
                    for (uint32_t i = tid; i < n_round; i += FT) dst[i] = items[i];
                    __syncthreads();
                }
            }
            run_f += tot & 0xFFFFu;
            run_r += tot >> 16;
        }
    } else {
        // Sparse PAM sites: warp per tile.  The CTA's 8 warps take 8 consecutive tiles per
        // round; each warp scans its tile's 256 word-pair masks (8 coalesced 16-byte loads
        // per lane, one warp scan per load), the tile totals are exchanged once per round
        // (two CTA barriers per 8 tiles instead of ~6 per tile), and every lane writes its
        // items straight to their ordered slots (L2 merges the partial sectors).
        constexpr int P2J = FT / 32;          // word-pair loads per lane and tile (8)
        unsigned long long run_f = 0, run_r = 0;
        const uint4* mptr = reinterpret_cast<const uint4*>(a.masks);
        for (uint32_t k = 0; k < n_mine; k += FT / 32) {
            const uint32_t tile = t_begin + k + (uint32_t)warp;
            const bool mine = k + (uint32_t)warp < n_mine;
            uint4 m[P2J];
            uint32_t off[P2J];                 // lane's exclusive offset in the tile per load (fwd | rev << 16)
            uint32_t acc = 0;                  // running tile total (fwd | rev << 16), warp-uniform
#pragma unroll
            for (int j = 0; j < P2J; j++)
                m[j] = mine ? __ldcg(mptr + (size_t)tile * FT + 32 * j + lane) : make_uint4(0, 0, 0, 0);
#pragma unroll
            for (int j = 0; j < P2J; j++) {
                const uint32_t c = (uint32_t)(__popc(m[j].x) + __popc(m[j].z)) |
                                   ((uint32_t)(__popc(m[j].y) + __popc(m[j].w)) << 16);
                uint32_t x = c;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
                    if (lane >= o) x += y;
                }
                off[j] = acc + x - c;
                acc += __shfl_sync(0xffffffffu, x, 31);
            }
            if (lane == 0) s_warp[warp] = acc;
            __syncthreads();
            unsigned long long bf = s_base[0] + run_f, br = s_base[1] + run_r;
#pragma unroll
            for (int w = 0; w < FT / 32; w++) {
                const uint32_t t = s_warp[w];
                if (w < warp) { bf += t & 0xFFFFu; br += t >> 16; }
                run_f += t & 0xFFFFu;
                run_r += t >> 16;
            }
            __syncthreads();   // s_warp is rewritten by the next round
            if (!mine) continue;
            const uint32_t pbase = tile * (uint32_t)FW * 32u + 64u * (uint32_t)lane;
#pragma unroll
            for (int j = 0; j < P2J; j++) {
                const uint32_t pj = pbase + 2048u * j;   // 32 lanes x 64 starts per load
#pragma unroll
                for (int st = 0; st < 2; st++) {
                    unsigned long long o = (st == 0 ? bf : br) + (st == 0 ? (off[j] & 0xFFFFu) : (off[j] >> 16));
                    uint32_t* out = a.out[st];
#pragma unroll
                    for (int w = 0; w < 2; w++) {
                        uint32_t mm = st == 0 ? (w ? m[j].z : m[j].x) : (w ? m[j].w : m[j].y);
                        while (mm) {
                            const int b = 31 - __clz(mm & (0u - mm));   // (one FLO; __ffs is BREV + FLO)
                            if (o < a.cap) out[o] = pj + 32u * w + (uint32_t)b;
                            o++;
                            mm &= mm - 1;
                        }
                    }
                }
            }
        }
    }
}

// per device (function attributes and occupancy are per-device state; several host threads
// may drive several GPUs, search_multi)
constexpr int FMAX_DEVICES = 64;
static int g_finder_blocks_per_sm[FMAX_DEVICES];
static int g_num_sms[FMAX_DEVICES];
static std::mutex g_finder_mu;

typedef void (*FinderFn)(FinderArgs);
template <bool VS, bool MO>
static FinderFn finder_fn_vs(uint32_t ne, bool wide) {
    if (wide) return cof_finder_kernel<-1, VS, MO, true>;   // L > 32: generic letter loop
    switch (ne) {
        case 0: return cof_finder_kernel<0, VS, MO, false>;
        case 1: return cof_finder_kernel<1, VS, MO, false>;
        case 2: return cof_finder_kernel<2, VS, MO, false>;
        case 3: return cof_finder_kernel<3, VS, MO, false>;
        case 4: return cof_finder_kernel<4, VS, MO, false>;
        case 5: return cof_finder_kernel<5, VS, MO, false>;
        case 6: return cof_finder_kernel<6, VS, MO, false>;
        default: return cof_finder_kernel<-1, VS, MO, false>;
    }
}
static FinderFn finder_fn(uint32_t ne, bool vs, bool masks_only = false, bool wide = false) {
    if (masks_only) return vs ? finder_fn_vs<true, true>(ne, wide) : finder_fn_vs<false, true>(ne, wide);
    return vs ? finder_fn_vs<true, false>(ne, wide) : finder_fn_vs<false, false>(ne, wide);
}

static cof_status finder_setup(int* bps_out, int* sms_out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return cuda_error(e, "finder setup");
    if (dev < 0 || dev >= FMAX_DEVICES) return set_error(COF_E_CUDA, "finder setup: device %d out of range", dev);
    std::lock_guard<std::mutex> lk(g_finder_mu);
    if (g_finder_blocks_per_sm[dev] <= 0) {
        int bps_min = 1 << 30;
        for (uint32_t k = 0; k < 64; k++) {
            FinderFn fn = finder_fn(k & 7, (k >> 3) & 1, (k >> 4) & 1, k >= 32);
            e = cudaFuncSetAttribute((const void*)fn, cudaFuncAttributeMaxDynamicSharedMemorySize, FSMEM);
            if (e != cudaSuccess) return cuda_error(e, "finder setup");
            int bps = 0;
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, (const void*)fn, FT, FSMEM);
            if (e != cudaSuccess) return cuda_error(e, "finder occupancy");
            if (bps < bps_min) bps_min = bps;
        }
        int sms = 0;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        g_num_sms[dev] = sms;
        g_finder_blocks_per_sm[dev] = bps_min > 0 ? bps_min : 1;
    }
    *bps_out = g_finder_blocks_per_sm[dev];
    *sms_out = g_num_sms[dev];
    return COF_OK;
}

}  // namespace cof

using namespace cof;

extern "C" {

size_t cof_find_workspace_bytes(uint64_t n_bases) {
    // per-CTA totals (at most FMAX_CTAS CTAs) + the grid barrier counter + 8 bytes of PAM
    // masks per plane word (the tiles cover cof_plane_words(n_bases) words)
    return FWS_MASKS + (size_t)cof_plane_words(n_bases) * 8;
}

}  // extern "C"

namespace cof {
// Shared by cof_find_pam (ordered item lists) and cof_find_compare (masks only).
cof_status find_launch(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                       uint32_t* items_fwd, uint32_t* items_rev, uint64_t items_cap, bool masks_only,
                       cudaStream_t stream);
}

extern "C" {

cof_status cof_find_pam(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                        uint32_t* items_fwd, uint32_t* items_rev, uint64_t items_cap, uint64_t* n_fwd,
                        uint64_t* n_rev, cof_stream s) {
    if (!plan || !plan_dev || !dev || !workspace || !items_fwd || !items_rev)
        return set_error(COF_E_ARG, "cof_find_pam: NULL argument");
    cudaStream_t stream = (cudaStream_t)s;
    cof_status st = find_launch(plan, plan_dev, dev, workspace, items_fwd, items_rev, items_cap, false, stream);
    if (st != COF_OK) return st;
    unsigned long long* counters = (unsigned long long*)((uint8_t*)plan_dev + plan->lay.counters);
    if (n_fwd || n_rev) {
        uint64_t c[2];
        cudaError_t e = cudaMemcpyAsync(c, counters, sizeof c, cudaMemcpyDeviceToHost, stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
        if (e != cudaSuccess) return cuda_error(e, "cof_find_pam counts");
        if (n_fwd) *n_fwd = c[0];
        if (n_rev) *n_rev = c[1];
        if (c[0] > items_cap || c[1] > items_cap)
            return set_error(COF_E_CAPACITY, "cof_find_pam: %llu/%llu items exceed capacity %llu",
                             (unsigned long long)c[0], (unsigned long long)c[1], (unsigned long long)items_cap);
    }
    return COF_OK;
}

}  // extern "C"

namespace cof {
const uint4* finder_masks(const void* workspace) {
    return reinterpret_cast<const uint4*>((const uint8_t*)workspace + FWS_MASKS);
}
uint64_t finder_word_pairs(const cof_plan* plan, const cof_chunk* dev) {
    const uint64_t L = plan->L;
    uint64_t limit = dev->n_bases >= L ? dev->n_bases - L + 1 : 0;
    if (!dev->n_segs && limit > dev->n_owned) limit = dev->n_owned;
    const uint64_t n_tiles = (limit + (uint64_t)FW * 32 - 1) / ((uint64_t)FW * 32);
    return n_tiles * FT;   // one uint4 {fwd0, rev0, fwd1, rev1} per thread-slot of every tile
}

cof_status find_launch(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                       uint32_t* items_fwd, uint32_t* items_rev, uint64_t items_cap, bool masks_only,
                       cudaStream_t stream) {
    if (!plan || !plan_dev || !dev || !workspace) return set_error(COF_E_ARG, "find: NULL argument");
    if (!dev->lo || !dev->hi || !dev->nm) return set_error(COF_E_ARG, "cof_find_pam: chunk planes are NULL");
    if (((uintptr_t)dev->lo | (uintptr_t)dev->hi | (uintptr_t)dev->nm | (uintptr_t)dev->vs) & 15)
        return set_error(COF_E_ARG, "cof_find_pam: planes must be 16-byte aligned");
    int f_bps = 0, f_sms = 0;
    cof_status st = finder_setup(&f_bps, &f_sms);
    if (st != COF_OK) return st;
    const uint64_t L = plan->L;
    if (dev->n_segs && !dev->vs) return set_error(COF_E_ARG, "cof_find_pam: multi-segment chunk without vs plane");
    if (dev->n_bases >= (1ull << 32)) return set_error(COF_E_ARG, "cof_find_pam: n_bases must be < 2^32");
    uint64_t limit = dev->n_bases >= L ? dev->n_bases - L + 1 : 0;
    if (!dev->n_segs && limit > dev->n_owned) limit = dev->n_owned;
    const uint32_t n_tiles = (uint32_t)((limit + (uint64_t)FW * 32 - 1) / ((uint64_t)FW * 32));
    unsigned long long* counters = (unsigned long long*)((uint8_t*)plan_dev + plan->lay.counters);
    cudaError_t e = cudaMemsetAsync(counters, 0, 2 * sizeof(uint64_t), stream);
    if (e == cudaSuccess && n_tiles)
        e = cudaMemsetAsync((uint8_t*)workspace + FWS_BARRIER, 0, 64, stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_find_pam memset");
    if (n_tiles) {
        FinderArgs a;
        a.lo = dev->lo; a.hi = dev->hi; a.nm = dev->nm;
        a.vs = dev->n_segs ? dev->vs : nullptr;
        a.limit = limit;
        a.out[0] = items_fwd; a.out[1] = items_rev;
        a.cap = items_cap;
        a.status = (uint64_t*)workspace;
        a.barrier = (unsigned int*)((uint8_t*)workspace + FWS_BARRIER);
        a.masks = (uint32_t*)((uint8_t*)workspace + FWS_MASKS);
        a.counters = counters;
        a.n_tiles = n_tiles;
        a.ne = plan->pam[0].n;
        {   // expected PAM sites per start and strand on a uniform genome: stage when dense
            double d = 1.0;
            for (uint32_t k = 0; k < plan->pam[0].n; k++) d *= __builtin_popcount(plan->pam[0].set[k]) / 4.0;
            a.stage = d >= 0.03 ? 1u : 0u;
        }
        bool wide = false;
        for (int st = 0; st < 2; st++)
            for (uint32_t k = 0; k < plan->pam[st].n; k++) wide |= plan->pam[st].j[k] >= 32;
        for (int st = 0; st < 2; st++)
            for (uint32_t k = 0; k < plan->pam[st].n; k++) {
                const uint32_t set = plan->pam[st].set[k];
                a.pj[st][k] = plan->pam[st].j[k];
                a.psel[st][k] = make_uint4(0u - (set & 1u), 0u - ((set >> 1) & 1u), 0u - ((set >> 2) & 1u),
                                           0u - ((set >> 3) & 1u));
            }
        uint32_t grid = (uint32_t)f_sms * (uint32_t)f_bps;
        if (grid > FMAX_CTAS) grid = FMAX_CTAS;
        if (grid > n_tiles) grid = n_tiles;
        FinderFn fn = finder_fn(a.ne, a.vs != nullptr, masks_only, wide);
        if (masks_only) {   // pass 1 only: no grid-wide exchange, a plain launch
            fn<<<grid, FT, FSMEM, stream>>>(a);
            e = cudaGetLastError();
        } else {
            // the grid exchange between pass 1 and pass 2 needs every CTA resident at once:
            // a cooperative launch guarantees it (or fails with
            // cudaErrorCooperativeLaunchTooLarge -> COF_E_CUDA) instead of hanging when other
            // work holds SMs; the grid never exceeds the occupancy limit computed above
            void* args[] = {(void*)&a};
            e = cudaLaunchCooperativeKernel((const void*)fn, dim3(grid), dim3(FT), args, FSMEM, stream);
        }
        if (e != cudaSuccess) return cuda_error(e, "cof_finder_kernel launch");
        count_launches(1);
    }
    return COF_OK;
}
}  // namespace cof
