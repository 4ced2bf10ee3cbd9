// Device decoration of sorted hit keys into output records (M10, on the GPU).
//
// Paper: the host "saves the results (chromosome number, position, direction, the number of
// mismatched bases and potential off-target DNA sequence with mismatched bases)".
// Host decoration (cof_collect) costs ~50-100 ns per hit on a CPU core; here one thread
// builds one 56-byte cof_hit from the device planes: the L-base window (three 32-bit plane
// slices), its mismatch mask against the guide in strand orientation (one-hot masks,
// bit-parallel), the site string read along the strand (reading G6) with mismatches
// lower-cased (G19), and the chunk coordinate mapped back to (chromosome, position)
// through the segment table.  Records leave in key order, so a sorted key buffer gives a
// sorted record buffer (G13).
#include <cuda_runtime.h>

#include "cof_internal.h"
#include "dev_common.cuh"

namespace cof {

struct DecorArgs {
    const uint32_t* lo;
    const uint32_t* hi;
    const uint32_t* nm;
    const unsigned long long* keys;
    uint64_t n;                 // host count, or ON_DEVICE: min(*count, cap)
    const unsigned long long* count;
    uint64_t cap;
    void* out;                  // cof_hit[] (L <= 32) or cof_hit64[]
    const unsigned long long* onehot;   // [2][n_guides][5] 64-bit window-offset masks
    const cof_segment* segs;    // device copy, n_segs entries (0: single segment)
    uint32_t n_segs;
    uint32_t n_guides;
    uint32_t L;
    uint32_t chrom;
    uint64_t start;
    unsigned int* bad;          // set to 1 if a key is inconsistent with the chunk / plan
};

template <typename HIT>
__device__ __forceinline__ void decorate_one(const DecorArgs& a, uint64_t i);

template <typename HIT>
__global__ void __launch_bounds__(256) cof_decorate_kernel(const __grid_constant__ DecorArgs a) {
    uint64_t n = a.n;
    if (a.count) {
        n = *a.count;
        if (n > a.cap) n = a.cap;
    }
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        decorate_one<HIT>(a, i);
}

// 64 consecutive bases from position p (bit j = base p+j); the third word only when needed.
__device__ __forceinline__ unsigned long long plane_window64(const uint32_t* __restrict__ plane, uint32_t p,
                                                             bool wide) {
    const uint32_t w = p >> 5, sh = p & 31;
    const uint32_t a = __ldg(plane + w), b = __ldg(plane + w + 1);
    const uint32_t c = wide ? __ldg(plane + w + 2) : 0u;
    return (unsigned long long)__funnelshift_r(a, b, sh) | ((unsigned long long)__funnelshift_r(b, c, sh) << 32);
}

template <typename HIT>
__device__ __forceinline__ void decorate_one(const DecorArgs& a, uint64_t i) {
    constexpr int MAXL = (int)sizeof(((HIT*)nullptr)->site) - 2;   // 32 or 64
    constexpr int NW = (int)sizeof(HIT) / 4;                          // record words
    const unsigned long long key = a.keys[i];
    const uint32_t pos = (uint32_t)(key >> 32);
    const uint32_t strand = (uint32_t)(key >> 31) & 1u;
    const uint32_t guide = (uint32_t)(key >> 7) & 0xFFFFFFu;
    const uint32_t mm = (uint32_t)key & 127u;
    const uint32_t L = a.L;
    bool ok = guide < a.n_guides;
    const uint32_t g = ok ? guide : 0u;
    // (a one-word window suffices while the window ends inside the second word)
    const bool wide = MAXL > 32 && (pos & 31u) + L > 32u;
    const unsigned long long lo = plane_window64(a.lo, pos, wide), hi = plane_window64(a.hi, pos, wide),
                             nm = plane_window64(a.nm, pos, wide);
    const unsigned long long* oh = a.onehot + ((size_t)strand * a.n_guides + g) * 5;
    const unsigned long long match = (~lo & ~hi & ~nm & __ldg(oh + 0)) | (lo & ~hi & ~nm & __ldg(oh + 1)) |
                                     (~lo & hi & ~nm & __ldg(oh + 2)) | (lo & hi & ~nm & __ldg(oh + 3));
    const unsigned long long mis = __ldg(oh + 4) & ~match;
    ok = ok && (uint32_t)__popcll(mis) == mm;
    // chromosome and position
    uint32_t chrom = a.chrom;
    unsigned long long cpos = a.start + pos;
    if (a.n_segs) {
        uint32_t lo_k = 0, hi_k = a.n_segs;
        while (hi_k - lo_k > 1) {
            const uint32_t mid = (lo_k + hi_k) >> 1;
            if (a.segs[mid].chunk_off <= pos) lo_k = mid;
            else hi_k = mid;
        }
        const cof_segment sg = a.segs[lo_k];
        ok = ok && pos >= sg.chunk_off && pos < sg.chunk_off + sg.n_owned;
        chrom = sg.chrom;
        cpos = sg.chrom_off + (pos - sg.chunk_off);
    }
    if (!ok) atomicOr(a.bad, 1u);
    // record: guide(4) chrom(4) pos(8) strand(1) mm(1) site(34 | 66) pad(4 | 4) = 56 | 88 bytes
    uint32_t w[NW];
    w[0] = guide;
    w[1] = chrom;
    w[2] = (uint32_t)cpos;
    w[3] = (uint32_t)(cpos >> 32);
    w[4] = (uint32_t)(strand ? '-' : '+') | (mm << 8);
#pragma unroll
    for (int k = 5; k < NW; k++) w[k] = 0;
    // site bytes start at byte offset 18 (word 4, byte 2)
#pragma unroll
    for (int j = 0; j < MAXL; j++) {
        if ((uint32_t)j < L) {
            const uint32_t k = strand ? L - 1 - (uint32_t)j : (uint32_t)j;
            uint32_t c = (((lo >> k) & 1u) | (((hi >> k) & 1u) << 1));
            if (strand) c ^= 3u;                       // complement: A<->T, C<->G
            const bool isn = (nm >> k) & 1u;
            const bool m = (mis >> k) & 1u;
            // "ACGT"[c] / 'N', lower-cased (| 0x20) when mismatched
            const uint32_t ch = (isn ? 0x4Eu : (0x54474341u >> (8 * c)) & 0xFFu) | (m ? 0x20u : 0u);
            const int byte = 18 + j;
            w[byte >> 2] |= ch << (8 * (byte & 3));
        }
    }
    uint2* dst = reinterpret_cast<uint2*>(reinterpret_cast<HIT*>(a.out) + i);
#pragma unroll
    for (int k = 0; k < NW / 2; k++) dst[k] = make_uint2(w[2 * k], w[2 * k + 1]);
}

}  // namespace cof

using namespace cof;

extern "C" {

size_t cof_decorate_workspace_bytes(uint32_t n_segs) {
    return 256 + (size_t)n_segs * sizeof(cof_segment);
}

}  // extern "C"

template <typename HIT>
static cof_status decorate_t(const char* fn, const cof_plan* plan, const void* plan_dev, const cof_chunk* dev,
                             const uint64_t* hits_dev, uint64_t n_hits, uint64_t cap, HIT* out_dev, void* workspace,
                             cof_stream s) {
    static_assert(sizeof(cof_hit) == 56 && sizeof(cof_hit64) == 88, "cof_hit layout");
    if (!plan || !plan_dev || !dev || !workspace || ((!hits_dev || !out_dev) && n_hits))
        return set_error(COF_E_ARG, "%s: NULL argument", fn);
    if (plan->L > sizeof out_dev->site - 2)   // cof_hit: L <= 32, cof_hit64: L <= 64
        return set_error(COF_E_ARG, "%s: L = %u does not fit the record (use cof_decorate64)", fn, plan->L);
    if (dev->n_segs && !dev->segs) return set_error(COF_E_ARG, "cof_decorate: multi-segment chunk without segs");
    cudaStream_t stream = (cudaStream_t)s;
    unsigned int* bad = (unsigned int*)workspace;
    cof_segment* dsegs = (cof_segment*)((uint8_t*)workspace + 256);
    cudaError_t e = cudaMemsetAsync(bad, 0, sizeof(unsigned int), stream);   // also for n_hits == 0
    if (e != cudaSuccess) return cuda_error(e, "cof_decorate");
    const bool on_dev = n_hits == COF_COUNT_ON_DEVICE;
    if (on_dev ? cap == 0 : n_hits == 0) return COF_OK;
    if (e == cudaSuccess && dev->n_segs)
        e = cudaMemcpyAsync(dsegs, dev->segs, (size_t)dev->n_segs * sizeof(cof_segment), cudaMemcpyHostToDevice, stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_decorate");
    DecorArgs a;
    a.lo = dev->lo; a.hi = dev->hi; a.nm = dev->nm;
    a.keys = (const unsigned long long*)hits_dev;
    a.n = on_dev ? 0 : n_hits;
    a.count = on_dev ? (const unsigned long long*)((const uint8_t*)plan_dev + plan->lay.counters + 16) : nullptr;
    a.cap = cap;
    a.out = out_dev;
    a.onehot = (const unsigned long long*)((const uint8_t*)plan_dev + plan->lay.onehot);
    a.segs = dsegs;
    a.n_segs = dev->n_segs;
    a.n_guides = plan->n_guides;
    a.L = plan->L;
    a.chrom = dev->chrom;
    a.start = dev->start;
    a.bad = bad;
    uint64_t blocks = ((on_dev ? cap : n_hits) + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;   // grid-stride beyond that
    cof_decorate_kernel<HIT><<<(uint32_t)blocks, 256, 0, stream>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "cof_decorate launch");
    count_launches(1);
    return COF_OK;
}

extern "C" {

cof_status cof_decorate(const cof_plan* plan, const void* plan_dev, const cof_chunk* dev, const uint64_t* hits_dev,
                        uint64_t n_hits, uint64_t cap, cof_hit* out_dev, void* workspace, cof_stream s) {
    return decorate_t("cof_decorate", plan, plan_dev, dev, hits_dev, n_hits, cap, out_dev, workspace, s);
}

cof_status cof_decorate64(const cof_plan* plan, const void* plan_dev, const cof_chunk* dev, const uint64_t* hits_dev,
                          uint64_t n_hits, uint64_t cap, cof_hit64* out_dev, void* workspace, cof_stream s) {
    return decorate_t("cof_decorate64", plan, plan_dev, dev, hits_dev, n_hits, cap, out_dev, workspace, s);
}

cof_status cof_decorate_check(const void* workspace, cof_stream s) {
    unsigned int bad = 0;
    cudaStream_t stream = (cudaStream_t)s;
    cudaError_t e = cudaMemcpyAsync(&bad, workspace, sizeof bad, cudaMemcpyDeviceToHost, stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    if (e != cudaSuccess) return cuda_error(e, "cof_decorate_check");
    if (bad) return set_error(COF_E_STATE, "cof_decorate: a hit key does not match the plan/chunk");
    return COF_OK;
}

}  // extern "C"
