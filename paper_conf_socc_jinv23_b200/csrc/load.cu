#include <omp.h>
#include <vector>
// Chunk load with the sparse planes built on the device (a2, host -> device).
//
// Paper: the host splits the genome into chunks and hands each to the device before the
// search kernel runs (Table III P:L84-L89 lists the buffer transfers).  Of the four
// planes of a chunk only lo/hi are dense: the N plane is a handful of runs (assembly gaps,
// rare IUPAC letters) and the valid-start plane of a multi-segment chunk is one interval
// per segment.  cof_load_chunk_runs copies lo/hi (1/4 B per base) and rebuilds nm and vs
// from their interval lists on the device, instead of moving 1/8 B per base for each over
// PCIe (the binding cost of the end-to-end path once the kernels are fast).
#include <algorithm>

#include <cuda_runtime.h>

#include "cof_internal.h"

namespace cof {

constexpr int RUNS_PER_LAUNCH = 256;   // intervals per launch, passed in the parameter space

struct FillArgs {
    uint32_t* nm;
    uint32_t* vs;          // or nullptr
    uint64_t words;        // cof_plane_words(n_bases)
    uint64_t n_bases;
};

// nm: 0 for every base, 1 past the last base (padding reads as N); vs: 0 everywhere.
__global__ void cof_fill_planes(const __grid_constant__ FillArgs a) {
    const uint64_t full = a.n_bases >> 5, rem = a.n_bases & 31;
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < a.words;
         w += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t v = 0;
        if (w > full || (w == full && rem == 0)) v = ~0u;
        else if (w == full) v = ~0u << rem;
        a.nm[w] = v;
        if (a.vs) a.vs[w] = 0u;
    }
}

struct RunArgs {
    uint32_t* plane;
    uint32_t n;
    ulonglong2 run[RUNS_PER_LAUNCH];   // [begin, end) bit ranges, disjoint
};

// One block per interval: full words are stored, the (at most two) partial words OR-ed in
// (two intervals may share a word).
__global__ void __launch_bounds__(256) cof_set_runs(const __grid_constant__ RunArgs a) {
    if (blockIdx.x >= a.n) return;
    const unsigned long long b = a.run[blockIdx.x].x, e = a.run[blockIdx.x].y;
    if (e <= b) return;
    const unsigned long long w0 = b >> 5, w1 = (e - 1) >> 5;
    for (unsigned long long w = w0 + threadIdx.x; w <= w1; w += blockDim.x) {
        uint32_t m = ~0u;
        if (w == w0) m &= ~0u << (uint32_t)(b & 31);
        if (w == w1 && (e & 31)) m &= ~0u >> (32u - (uint32_t)(e & 31));
        if (m == ~0u) a.plane[w] = m;
        else atomicOr(a.plane + w, m);
    }
}

static cof_status set_runs(uint32_t* plane, const uint64_t* runs, uint64_t n, cudaStream_t s) {
    static thread_local RunArgs R;
    for (uint64_t i = 0; i < n; i += RUNS_PER_LAUNCH) {
        R.plane = plane;
        R.n = (uint32_t)std::min<uint64_t>(RUNS_PER_LAUNCH, n - i);
        for (uint32_t k = 0; k < R.n; k++) R.run[k] = make_ulonglong2(runs[2 * (i + k)], runs[2 * (i + k) + 1]);
        cof_set_runs<<<R.n, 256, 0, s>>>(R);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "cof_set_runs launch");
        count_launches(1);
    }
    return COF_OK;
}

}  // namespace cof

using namespace cof;

extern "C" {

// N runs of words [w0, w1) of an nm plane (bases < n_bases only), appended to out.
static void n_runs_range(const uint32_t* nm, uint64_t n_bases, uint64_t w0, uint64_t w1,
                         std::vector<uint64_t>& out) {
    bool open = false;
    uint64_t begin = 0;
    const uint64_t words = (n_bases + 31) / 32;
    for (uint64_t w = w0; w < w1; w++) {
        uint32_t v = nm[w];
        if (w == words - 1 && (n_bases & 31)) v &= ~0u >> (32 - (n_bases & 31));   // bases only
        if (!open && v == 0) continue;
        if (open && v == ~0u && (w < words - 1 || !(n_bases & 31))) continue;
        for (uint32_t bit = 0; bit < 32; bit++) {      // a word with an edge: bit by bit
            const uint64_t p = w * 32 + bit;
            if (p >= n_bases) break;
            const bool isn = (v >> bit) & 1u;
            if (isn && !open) { open = true; begin = p; }
            else if (!isn && open) {
                out.push_back(begin);
                out.push_back(p);
                open = false;
            }
        }
    }
    if (open) {
        out.push_back(begin);
        out.push_back(std::min<uint64_t>(w1 * 32, n_bases));
    }
}

cof_status cof_n_runs(const uint32_t* nm, uint64_t n_bases, uint64_t* runs, uint64_t cap, uint64_t* n_runs) {
    if (!nm || !n_runs || (!runs && cap)) return set_error(COF_E_ARG, "cof_n_runs: NULL argument");
    // word ranges scanned in parallel; a run cut by a range boundary is joined afterwards
    const uint64_t words = (n_bases + 31) / 32;
    const int nt = words > (1u << 20) ? std::max(1, omp_get_max_threads()) : 1;
    std::vector<std::vector<uint64_t>> part(nt);
    const uint64_t per = (words + nt - 1) / nt;
#pragma omp parallel for schedule(static) num_threads(nt) if (nt > 1)
    for (int t = 0; t < nt; t++)
        n_runs_range(nm, n_bases, std::min(words, t * per), std::min(words, (t + 1) * per), part[t]);
    uint64_t n = 0, last_end = ~0ull;
    for (int t = 0; t < nt; t++) {
        for (size_t k = 0; k < part[t].size(); k += 2) {
            const uint64_t b = part[t][k], e = part[t][k + 1];
            if (n && b == last_end) {                  // continues the previous range's run
                if (n <= cap) runs[2 * (n - 1) + 1] = e;
            } else {
                if (n < cap) { runs[2 * n] = b; runs[2 * n + 1] = e; }
                n++;
            }
            last_end = e;
        }
    }
    *n_runs = n;
    if (n > cap) return set_error(COF_E_CAPACITY, "cof_n_runs: %llu runs exceed capacity %llu",
                                  (unsigned long long)n, (unsigned long long)cap);
    return COF_OK;
}

static cof_status load_runs(const cof_chunk* host, const uint64_t* runs, uint64_t n_runs, cof_chunk* dev,
                            cudaStream_t st, cudaStream_t fs) {
    if (!host || !dev || !host->lo || !host->hi || !dev->lo || !dev->hi || !dev->nm || (!runs && n_runs))
        return set_error(COF_E_ARG, "cof_load_chunk_runs: NULL argument");
    if (host->n_segs && (!host->segs || !dev->vs))
        return set_error(COF_E_ARG, "cof_load_chunk_runs: multi-segment chunk needs segs and a device vs plane");
    for (uint64_t i = 0; i < n_runs; i++)
        if (runs[2 * i] > runs[2 * i + 1] || runs[2 * i + 1] > host->n_bases || (i && runs[2 * i] < runs[2 * i - 1]))
            return set_error(COF_E_ARG, "cof_load_chunk_runs: run %llu is not an ascending interval inside the chunk",
                             (unsigned long long)i);
    const uint64_t words = cof_plane_words(host->n_bases);
    const size_t bytes = words * sizeof(uint32_t);
    cudaError_t e;
    if ((e = cudaMemcpyAsync(dev->lo, host->lo, bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess ||
        (e = cudaMemcpyAsync(dev->hi, host->hi, bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_error(e, "cof_load_chunk_runs");
    FillArgs f{dev->nm, host->n_segs ? dev->vs : nullptr, words, host->n_bases};
    const uint64_t blocks = std::min<uint64_t>((words + 255) / 256, 148 * 8);
    cof_fill_planes<<<(uint32_t)std::max<uint64_t>(blocks, 1), 256, 0, fs>>>(f);
    if ((e = cudaGetLastError()) != cudaSuccess) return cuda_error(e, "cof_fill_planes launch");
    count_launches(1);
    cof_status r = set_runs(dev->nm, runs, n_runs, fs);
    if (r != COF_OK) return r;
    if (host->n_segs) {
        std::vector<uint64_t> own(2 * (size_t)host->n_segs);
        for (uint32_t k = 0; k < host->n_segs; k++) {
            const cof_segment& g = host->segs[k];
            if (g.chunk_off + g.n_owned > host->n_bases)
                return set_error(COF_E_ARG, "cof_load_chunk_runs: segment %u leaves the chunk", k);
            own[2 * k] = g.chunk_off;
            own[2 * k + 1] = g.chunk_off + g.n_owned;
        }
        r = set_runs(dev->vs, own.data(), host->n_segs, fs);
        if (r != COF_OK) return r;
    }
    dev->chrom = host->chrom;
    dev->n_segs = host->n_segs;
    dev->start = host->start;
    dev->n_bases = host->n_bases;
    dev->n_owned = host->n_owned;
    dev->segs = host->segs;
    if (!host->n_segs) dev->vs = nullptr;
    return COF_OK;
}

cof_status cof_load_chunk_runs(const cof_chunk* host, const uint64_t* runs, uint64_t n_runs, cof_chunk* dev,
                               cof_stream s) {
    return load_runs(host, runs, n_runs, dev, (cudaStream_t)s, (cudaStream_t)s);
}

cof_status cof_load_chunk_runs_split(const cof_chunk* host, const uint64_t* runs, uint64_t n_runs, cof_chunk* dev,
                                     cof_stream s_copy, cof_stream s_fill) {
    return load_runs(host, runs, n_runs, dev, (cudaStream_t)s_copy, (cudaStream_t)s_fill);
}

}  // extern "C"
