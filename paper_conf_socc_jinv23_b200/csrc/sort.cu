// Deterministic ordering of hit keys (K3, M10) for sm_100a: stable LSD radix sort.
//
// Paper: hit slots come from an atomic counter and "the order of updates is not
// deterministic" (Listing 1).  Reading G13 fixes the output order
// to (chromosome, position, '+' before '-', guide).  Within a chunk the key
//   key = pos << 32 | strand << 31 | guide << 7 | mm
// orders exactly that way; only the bits that can vary are sorted: the compressed key
//   k' = pos << (GB + 1) | strand << GB | guide      (GB = bits of the largest guide index)
// is cut into 8-bit digits, one pass per digit.  Each pass: per-tile digit histograms
// (shared-memory atomics) + digit totals, a per-digit scan over tiles (one CTA per digit), and a
// stable scatter that ranks keys inside a tile with __match_any_sync in index order.
#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"

namespace cof {

constexpr int ST = 256;             // threads per CTA
constexpr int SV = 16;              // keys per thread per tile
constexpr int STILE = ST * SV;      // 4096 keys per tile

struct SortPass {
    const unsigned long long* src;
    unsigned long long* dst;
    uint32_t* hist;                 // [256][cap_tiles]
    uint32_t* totals;               // [256] keys per digit (zeroed before the pass)
    const unsigned long long* count;  // device count (n_hits) or nullptr
    uint64_t n_host;                // used when count == nullptr
    uint64_t cap;
    uint32_t cap_tiles;
    uint32_t shift;                 // digit position in k'
    uint32_t gb;                    // guide bits
};

__device__ __forceinline__ uint64_t sort_n(const SortPass& p) {
    uint64_t n = p.count ? (uint64_t)*p.count : p.n_host;
    return n < p.cap ? n : p.cap;
}

__device__ __forceinline__ uint32_t digit_of(unsigned long long key, uint32_t gb, uint32_t shift) {
    const uint64_t pos = key >> 32;
    const uint64_t strand = (key >> 31) & 1ull;
    const uint64_t guide = (key >> 7) & ((1ull << gb) - 1ull);
    const uint64_t kc = (pos << (gb + 1)) | (strand << gb) | guide;
    return (uint32_t)(kc >> shift) & 255u;
}

__global__ void __launch_bounds__(ST) cof_sort_hist(const __grid_constant__ SortPass p) {
    __shared__ uint32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t n = sort_n(p);
    const uint64_t base = (uint64_t)blockIdx.x * STILE;
    if (base < n) {
        unsigned long long kk[SV];
#pragma unroll
        for (int v = 0; v < SV; v++) {
            const uint64_t i = base + (uint64_t)v * ST + threadIdx.x;
            kk[v] = i < n ? __ldcg(p.src + i) : 0ull;
        }
#pragma unroll
        for (int v = 0; v < SV; v++) {
            const uint64_t i = base + (uint64_t)v * ST + threadIdx.x;
            if (i < n) atomicAdd(&h[digit_of(kk[v], p.gb, p.shift)], 1u);
        }
    }
    __syncthreads();
    p.hist[(size_t)threadIdx.x * p.cap_tiles + blockIdx.x] = h[threadIdx.x];
    if (h[threadIdx.x]) atomicAdd(&p.totals[threadIdx.x], h[threadIdx.x]);
}

// Offsets: CTA d turns row d of the [256][cap_tiles] histogram into global offsets
// (exclusive scan over tiles + the number of keys with a smaller digit).
__global__ void __launch_bounds__(ST) cof_sort_scan(const __grid_constant__ SortPass p) {
    __shared__ uint32_t s_warp[ST / 32];
    __shared__ uint32_t s_carry;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t d = blockIdx.x;
    uint32_t below = tid < (int)d ? p.totals[tid] : 0u;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) below += __shfl_xor_sync(0xffffffffu, below, o);
    if (lane == 0) s_warp[warp] = below;
    __syncthreads();
    if (tid == 0) {
        uint32_t b = 0;
        for (int w = 0; w < ST / 32; w++) b += s_warp[w];
        s_carry = b;
    }
    __syncthreads();
    uint32_t* row = p.hist + (size_t)d * p.cap_tiles;
    const uint32_t m = p.cap_tiles;
    for (uint32_t c0 = 0; c0 < m; c0 += ST * 4) {
        uint32_t v[4], sum = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t i = c0 + (uint32_t)tid * 4 + k;
            v[k] = i < m ? row[i] : 0u;
            sum += v[k];
        }
        uint32_t x = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        __syncthreads();
        if (lane == 31) s_warp[warp] = x;
        __syncthreads();
        if (warp == 0) {
            const uint32_t wv = lane < ST / 32 ? s_warp[lane] : 0u;
            uint32_t wi = wv;
#pragma unroll
            for (int o = 1; o < ST / 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, wi, o);
                if (lane >= o) wi += y;
            }
            if (lane < ST / 32) s_warp[lane] = wi - wv;
        }
        __syncthreads();
        uint32_t run = s_carry + s_warp[warp] + x - sum;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t i = c0 + (uint32_t)tid * 4 + k;
            if (i < m) row[i] = run;
            run += v[k];
        }
        __syncthreads();
        if (tid == ST - 1) s_carry = run;
        __syncthreads();
    }
}

// Stable scatter of one 4096-key tile.  Warp w owns keys [w*512, w*512+512) of the tile,
// lane l holds slots k = 0..15 (index w*512 + 32k + l, coalesced): going slot by slot with
// __match_any_sync and a warp-private digit counter gives every key its rank among the
// equal-digit keys of its warp in index order (no block barrier per slot).  One block-wide
// prefix then turns (warp, digit) counts into tile-local digit starts; keys are staged in
// shared memory in digit order and written out with consecutive threads writing
// consecutive keys of a digit run (coalesced).
__global__ void __launch_bounds__(ST) cof_sort_scatter(const __grid_constant__ SortPass p) {
    constexpr int NW = ST / 32;
    __shared__ uint32_t s_cnt[NW][256];          // per-warp digit counts -> exclusive prefixes
    __shared__ uint32_t s_goff[256];             // global offset of this tile's digit d
    __shared__ uint32_t s_dstart[256];           // tile-local start of digit d
    __shared__ uint32_t s_warp[NW];
    __shared__ unsigned long long s_keys[STILE];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint64_t n = sort_n(p);
    const uint64_t base = (uint64_t)blockIdx.x * STILE;
    if (base >= n) return;
    const uint32_t n_tile = (uint32_t)min((uint64_t)STILE, n - base);
#pragma unroll
    for (int w = 0; w < NW; w++) s_cnt[w][tid] = 0;
    s_goff[tid] = p.hist[(size_t)tid * p.cap_tiles + blockIdx.x];
    __syncthreads();

    unsigned long long key[SV];
    uint32_t rank[SV];
#pragma unroll
    for (int k = 0; k < SV; k++) {   // all loads first: 16 independent requests in flight
        const uint32_t li = (uint32_t)warp * (STILE / NW) + (uint32_t)k * 32 + lane;
        key[k] = li < n_tile ? __ldcs(p.src + base + li) : 0ull;
    }
#pragma unroll
    for (int k = 0; k < SV; k++) {
        const uint32_t li = (uint32_t)warp * (STILE / NW) + (uint32_t)k * 32 + lane;
        const bool ok = li < n_tile;
        const uint32_t d = ok ? digit_of(key[k], p.gb, p.shift) : 256u;
        const unsigned peers = __match_any_sync(0xffffffffu, d);
        const int leader = __ffs(peers) - 1;
        uint32_t old = 0;
        if (lane == leader && ok) old = s_cnt[warp][d];
        old = __shfl_sync(0xffffffffu, old, leader);
        if (lane == leader && ok) s_cnt[warp][d] = old + (uint32_t)__popc(peers);
        __syncwarp();
        rank[k] = old + (uint32_t)__popc(peers & lanemask_lt());
    }
    __syncthreads();
    // digit tid: exclusive prefix over warps, then exclusive scan of the digit totals
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < NW; w++) {
        const uint32_t c = s_cnt[w][tid];
        s_cnt[w][tid] = run;
        run += c;
    }
    uint32_t x = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) s_warp[warp] = x;
    __syncthreads();
    uint32_t wbase = 0;
#pragma unroll
    for (int w = 0; w < NW; w++) wbase += w < warp ? s_warp[w] : 0u;
    s_dstart[tid] = wbase + x - run;
    __syncthreads();
#pragma unroll
    for (int k = 0; k < SV; k++) {
        const uint32_t li = (uint32_t)warp * (STILE / NW) + (uint32_t)k * 32 + lane;
        if (li < n_tile) {
            const uint32_t d = digit_of(key[k], p.gb, p.shift);
            s_keys[s_dstart[d] + s_cnt[warp][d] + rank[k]] = key[k];
        }
    }
    __syncthreads();
    for (uint32_t j = tid; j < n_tile; j += ST) {
        const unsigned long long kk = s_keys[j];
        const uint32_t d = digit_of(kk, p.gb, p.shift);
        p.dst[s_goff[d] + (j - s_dstart[d])] = kk;
    }
}

__global__ void cof_sort_copy(const __grid_constant__ SortPass p) {
    const uint64_t n = sort_n(p);
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p.dst[i] = p.src[i];
}

static uint32_t bits_for(uint64_t x) {   // number of bits to represent values 0..x
    uint32_t b = 0;
    while (b < 64 && (x >> b)) b++;
    return b;
}

}  // namespace cof

using namespace cof;

extern "C" {

size_t cof_sort_workspace_bytes(uint64_t cap) {
    uint64_t tiles = (cap + STILE - 1) / STILE;
    if (!tiles) tiles = 1;
    return (size_t)(256 * tiles * sizeof(uint32_t) + 256 * sizeof(uint32_t));
}

cof_status cof_sort_hits(const cof_plan* plan, void* plan_dev, const cof_chunk* dev, uint64_t* hits, uint64_t* tmp,
                         uint64_t cap, uint64_t n_hits, void* workspace, cof_stream s) {
    if (!plan || !plan_dev || !dev || ((!hits || !tmp || !workspace) && cap))
        return set_error(COF_E_ARG, "cof_sort_hits: NULL argument");
    if (cap == 0) return COF_OK;
    cudaStream_t stream = (cudaStream_t)s;
    SortPass p;
    p.hist = (uint32_t*)workspace;
    p.count = n_hits == COF_COUNT_ON_DEVICE
                  ? (const unsigned long long*)((uint8_t*)plan_dev + plan->lay.counters + 2 * sizeof(uint64_t))
                  : nullptr;
    p.n_host = n_hits == COF_COUNT_ON_DEVICE ? 0 : n_hits;
    if (!p.count && p.n_host <= 1) return COF_OK;
    p.cap = cap;
    uint64_t eff = p.count ? cap : (p.n_host < cap ? p.n_host : cap);
    p.cap_tiles = (uint32_t)((eff + STILE - 1) / STILE);
    p.gb = bits_for(plan->n_guides - 1);
    const uint32_t pb = bits_for(dev->n_bases ? dev->n_bases - 1 : 0);   // positions are < n_bases
    const uint32_t total_bits = pb + 1 + p.gb;
    const uint32_t passes = (total_bits + 7) / 8;
    unsigned long long* a = (unsigned long long*)hits;
    unsigned long long* b = (unsigned long long*)tmp;
    p.totals = p.hist + (size_t)256 * p.cap_tiles;
    for (uint32_t k = 0; k < passes; k++) {
        p.src = a; p.dst = b; p.shift = 8 * k;
        cudaMemsetAsync(p.totals, 0, 256 * sizeof(uint32_t), stream);
        cof_sort_hist<<<p.cap_tiles, ST, 0, stream>>>(p);
        cof_sort_scan<<<256, ST, 0, stream>>>(p);
        cof_sort_scatter<<<p.cap_tiles, ST, 0, stream>>>(p);
        count_launches(3);
        unsigned long long* t = a; a = b; b = t;
    }
    if (a != (unsigned long long*)hits) {
        p.src = a; p.dst = (unsigned long long*)hits;
        cof_sort_copy<<<1184, 256, 0, stream>>>(p);
        count_launches(1);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "cof_sort_hits launch");
    return COF_OK;
}

}  // extern "C"
