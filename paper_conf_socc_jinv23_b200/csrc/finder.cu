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
// IUPAC set, AND-ed over letters.  Passing starts are compacted in order: CTA scan of the
// per-thread popcounts, single-pass decoupled look-back across tiles for the global
// offset, staging in shared memory and coalesced stores.  Bytes per base: 3/8 read +
// 4 x items written.
#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"

namespace cof {

constexpr int FT = 256;          // threads per CTA; one plane word per thread per tile
constexpr int FW = 256;          // words per tile (8192 window starts)
constexpr int FSTAGES = 4;       // TMA ring depth
constexpr int FLOAD = FW + 4;    // words per plane per stage: tile + halo, 16-byte multiple
constexpr uint32_t FSMEM = FSTAGES * 3 * FLOAD * 4 + FSTAGES * 8 + FW * 32 * 4;

struct FinderArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    uint64_t limit;              // valid window starts are [0, limit)
    uint32_t* out[2];            // '+' / '-' item lists
    uint64_t cap;
    uint64_t* status;            // workspace: one look-back word per tile (zeroed)
    unsigned long long* counters;  // plan_dev counters: [0] n_fwd, [1] n_rev
    uint32_t n_tiles;
    PamStrand pam[2];
};

// Membership of each of 32 bases (bit-parallel) in the IUPAC set `set` (A=1 C=2 G=4 T=8):
// a multiplexer on the 2-bit code selects the set bit; N (nm=1) is in no set (G2).
__device__ __forceinline__ uint32_t member(uint32_t lo, uint32_t hi, uint32_t nm, uint32_t set) {
    const uint32_t sA = 0u - (set & 1u), sC = 0u - ((set >> 1) & 1u);
    const uint32_t sG = 0u - ((set >> 2) & 1u), sT = 0u - ((set >> 3) & 1u);
    const uint32_t t0 = (hi & sG) | (~hi & sA);      // lo = 0: A or G
    const uint32_t t1 = (hi & sT) | (~hi & sC);      // lo = 1: C or T
    const uint32_t r = (lo & t1) | (~lo & t0);
    return r & ~nm;
}

constexpr uint64_t LB_AGG = 1ull << 62, LB_INC = 2ull << 62, LB_VAL = (1ull << 62) - 1;

__global__ void __launch_bounds__(FT) cof_finder_kernel(const __grid_constant__ FinderArgs a) {
    extern __shared__ __align__(128) uint8_t smem[];
    uint32_t* stage = reinterpret_cast<uint32_t*>(smem);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + FSTAGES * 3 * FLOAD * 4);
    uint32_t* items = reinterpret_cast<uint32_t*>(bars + FSTAGES);
    __shared__ uint32_t s_warp[FT / 32];
    __shared__ uint32_t s_tile_tot;
    __shared__ uint64_t s_prefix;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        for (int s = 0; s < FSTAGES; s++) mbar_init(&bars[s], 1);
        fence_mbar_init();
    }
    __syncthreads();

    auto issue = [&](uint32_t tile, int s) {
        const size_t w0 = (size_t)tile * FW;
        mbar_arrive_expect_tx(&bars[s], 3 * FLOAD * 4);
        bulk_g2s(stage + (s * 3 + 0) * FLOAD, a.lo + w0, FLOAD * 4, &bars[s]);
        bulk_g2s(stage + (s * 3 + 1) * FLOAD, a.hi + w0, FLOAD * 4, &bars[s]);
        bulk_g2s(stage + (s * 3 + 2) * FLOAD, a.nm + w0, FLOAD * 4, &bars[s]);
    };
    if (tid == 0) {
        for (int s = 0; s < FSTAGES; s++) {
            uint32_t t = blockIdx.x + (uint32_t)s * gridDim.x;
            if (t < a.n_tiles) issue(t, s);
        }
    }

    uint32_t it = 0;
    for (uint32_t tile = blockIdx.x; tile < a.n_tiles; tile += gridDim.x, it++) {
        const int s = (int)(it % FSTAGES);
        mbar_wait_parity(&bars[s], (it / FSTAGES) & 1u);
        const uint32_t* Slo = stage + (s * 3 + 0) * FLOAD;
        const uint32_t* Shi = stage + (s * 3 + 1) * FLOAD;
        const uint32_t* Snm = stage + (s * 3 + 2) * FLOAD;
        const uint32_t lo0 = Slo[tid], lo1 = Slo[tid + 1];
        const uint32_t hi0 = Shi[tid], hi1 = Shi[tid + 1];
        const uint32_t nm0 = Snm[tid], nm1 = Snm[tid + 1];

        const uint64_t p0 = ((uint64_t)tile * FW + tid) * 32;
        uint32_t valid;
        if (p0 >= a.limit) valid = 0;
        else if (a.limit - p0 >= 32) valid = ~0u;
        else valid = (1u << (uint32_t)(a.limit - p0)) - 1u;

        uint32_t m[2];
#pragma unroll
        for (int st = 0; st < 2; st++) {
            uint32_t acc = valid;
            const uint32_t n = a.pam[st].n;
            for (uint32_t e = 0; e < n; e++) {
                const uint32_t j = a.pam[st].j[e];
                const uint32_t l = __funnelshift_r(lo0, lo1, j);
                const uint32_t h = __funnelshift_r(hi0, hi1, j);
                const uint32_t x = __funnelshift_r(nm0, nm1, j);
                acc &= member(l, h, x, a.pam[st].set[e]);
            }
            m[st] = acc;
        }
        __syncthreads();   // every thread has read stage s: refill it
        if (tid == 0) {
            const uint32_t nt = tile + FSTAGES * gridDim.x;
            if (nt < a.n_tiles) {
                fence_proxy_async_smem();
                issue(nt, s);
            }
        }

        // ---- CTA exclusive scan of packed counts (fwd in bits 0..15, rev in 16..31)
        const uint32_t cnt = (uint32_t)__popc(m[0]) | ((uint32_t)__popc(m[1]) << 16);
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
            if (lane < FT / 32) s_warp[lane] = wi - wv;          // exclusive warp offsets
            const uint32_t tot = __shfl_sync(0xffffffffu, wi, FT / 32 - 1);
            // ---- decoupled look-back over tiles (values: fwd bits 0..30, rev bits 31..61)
            const uint64_t agg = (uint64_t)(tot & 0xFFFFu) | ((uint64_t)(tot >> 16) << 31);
            uint64_t excl = 0;
            if (tile == 0) {
                if (lane == 0) st_relaxed_gpu(&a.status[0], LB_INC | agg);
            } else {
                if (lane == 0) st_relaxed_gpu(&a.status[tile], LB_AGG | agg);
                int64_t pred = (int64_t)tile - 1;
                while (true) {
                    const int64_t idx = pred - lane;
                    const uint64_t v = idx >= 0 ? ld_relaxed_gpu(&a.status[idx]) : LB_INC;
                    const uint32_t flag = (uint32_t)(v >> 62);
                    if (__any_sync(0xffffffffu, flag == 0)) continue;
                    const uint32_t inc = __ballot_sync(0xffffffffu, flag == 2);
                    uint64_t val = v & LB_VAL;
                    if (inc) {
                        const int first = __ffs(inc) - 1;
                        if (lane > first) val = 0;
                    }
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) val += __shfl_xor_sync(0xffffffffu, val, o);
                    excl += val;
                    if (inc) break;
                    pred -= 32;
                }
                if (lane == 0) st_relaxed_gpu(&a.status[tile], LB_INC | (excl + agg));
            }
            if (lane == 0) {
                s_prefix = excl;
                s_tile_tot = tot;
                if (tile == a.n_tiles - 1) {
                    const uint64_t inc_all = excl + agg;
                    a.counters[0] = inc_all & 0x7FFFFFFFull;
                    a.counters[1] = (inc_all >> 31) & 0x7FFFFFFFull;
                }
            }
        }
        __syncthreads();
        const uint32_t local = s_warp[warp] + x - cnt;    // exclusive, packed
        const uint64_t pre = s_prefix;
        const uint32_t tot = s_tile_tot;

        // ---- ordered, coalesced output per strand through the shared staging buffer
#pragma unroll
        for (int st = 0; st < 2; st++) {
            uint32_t off = st == 0 ? (local & 0xFFFFu) : (local >> 16);
            uint32_t mm = m[st];
            const uint32_t pbase = (uint32_t)p0;
            while (mm) {
                const int b = __ffs(mm) - 1;
                items[off++] = pbase + (uint32_t)b;
                mm &= mm - 1;
            }
            __syncthreads();
            const uint32_t total = st == 0 ? (tot & 0xFFFFu) : (tot >> 16);
            const uint64_t base = st == 0 ? (pre & 0x7FFFFFFFull) : ((pre >> 31) & 0x7FFFFFFFull);
            uint32_t* out = a.out[st];
            for (uint32_t i = tid; i < total; i += FT) {
                const uint64_t o = base + i;
                if (o < a.cap) out[o] = items[i];
            }
            __syncthreads();
        }
    }
}

static int g_finder_blocks_per_sm = -1;
static int g_num_sms = -1;

static cof_status finder_setup() {
    if (g_finder_blocks_per_sm > 0) return COF_OK;
    cudaError_t e = cudaFuncSetAttribute(cof_finder_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, FSMEM);
    if (e != cudaSuccess) return cuda_error(e, "finder setup");
    int dev = 0, sms = 0, bps = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cof_finder_kernel, FT, FSMEM);
    if (e != cudaSuccess) return cuda_error(e, "finder occupancy");
    g_num_sms = sms;
    g_finder_blocks_per_sm = bps > 0 ? bps : 1;
    return COF_OK;
}

}  // namespace cof

using namespace cof;

extern "C" {

size_t cof_find_workspace_bytes(uint64_t n_owned) {
    uint64_t tiles = (n_owned + (uint64_t)FW * 32 - 1) / ((uint64_t)FW * 32);
    return (size_t)(tiles ? tiles : 1) * sizeof(uint64_t);
}

cof_status cof_find_pam(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, void* workspace,
                        uint32_t* items_fwd, uint32_t* items_rev, uint64_t items_cap, uint64_t* n_fwd,
                        uint64_t* n_rev, cof_stream s) {
    if (!plan || !plan_dev || !dev || !workspace || !items_fwd || !items_rev)
        return set_error(COF_E_ARG, "cof_find_pam: NULL argument");
    if (!dev->lo || !dev->hi || !dev->nm) return set_error(COF_E_ARG, "cof_find_pam: chunk planes are NULL");
    if (dev->n_owned >= (1ull << 31)) return set_error(COF_E_ARG, "cof_find_pam: n_owned must be < 2^31");
    if (((uintptr_t)dev->lo | (uintptr_t)dev->hi | (uintptr_t)dev->nm) & 15)
        return set_error(COF_E_ARG, "cof_find_pam: planes must be 16-byte aligned");
    cof_status st = finder_setup();
    if (st != COF_OK) return st;
    cudaStream_t stream = (cudaStream_t)s;
    const uint64_t L = plan->L;
    uint64_t limit = dev->n_bases >= L ? dev->n_bases - L + 1 : 0;
    if (limit > dev->n_owned) limit = dev->n_owned;
    const uint32_t n_tiles = (uint32_t)((limit + (uint64_t)FW * 32 - 1) / ((uint64_t)FW * 32));
    unsigned long long* counters = (unsigned long long*)((uint8_t*)plan_dev + plan->lay.counters);
    cudaError_t e = cudaMemsetAsync(counters, 0, 2 * sizeof(uint64_t), stream);
    if (e == cudaSuccess && n_tiles)
        e = cudaMemsetAsync(workspace, 0, (size_t)n_tiles * sizeof(uint64_t), stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_find_pam memset");
    if (n_tiles) {
        FinderArgs a;
        a.lo = dev->lo; a.hi = dev->hi; a.nm = dev->nm;
        a.limit = limit;
        a.out[0] = items_fwd; a.out[1] = items_rev;
        a.cap = items_cap;
        a.status = (uint64_t*)workspace;
        a.counters = counters;
        a.n_tiles = n_tiles;
        a.pam[0] = plan->pam[0];
        a.pam[1] = plan->pam[1];
        uint32_t grid = (uint32_t)g_num_sms * (uint32_t)g_finder_blocks_per_sm;
        if (grid > n_tiles) grid = n_tiles;
        cof_finder_kernel<<<grid, FT, FSMEM, stream>>>(a);
        e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "cof_finder_kernel launch");
        count_launches(1);
    }
    if (n_fwd || n_rev) {
        uint64_t c[2];
        e = cudaMemcpyAsync(c, counters, sizeof c, cudaMemcpyDeviceToHost, stream);
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
