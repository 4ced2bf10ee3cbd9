// Plan creation (M1): pattern + guides + thresholds -> PAM strands for the finder and the
// device image of the guide tables for the comparer.  Host-only, no CUDA kernels.
//
// Paper: the input specification ("the desired pattern, query sequences, and
// maximum mismatch number"); the comparer's query arrays comp/comp_index hold the query
// and its reverse-complement ("two patterns from which one is selected based on the
// value of a flag"; Listing 1).  Here both orientations are
// prepared once on the host for every guide.
#include <algorithm>
#include <cstring>
#include <map>

#include <cuda_runtime.h>

#include "cof_internal.h"

namespace cof {

uint8_t iupac_mask(char c) {
    switch (c >= 'a' && c <= 'z' ? c - 32 : c) {
        case 'A': return 1;  case 'C': return 2;  case 'G': return 4;  case 'T': return 8;
        case 'R': return 1 | 4;   case 'Y': return 2 | 8;   case 'S': return 2 | 4;
        case 'W': return 1 | 8;   case 'K': return 4 | 8;   case 'M': return 1 | 2;
        case 'B': return 2 | 4 | 8;  case 'D': return 1 | 4 | 8;  case 'H': return 1 | 2 | 8;
        case 'V': return 1 | 2 | 4;  case 'N': return 15;
        default: return 0;
    }
}

static size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

}  // namespace cof

using namespace cof;

extern "C" {

cof_status cof_plan_create(const char* pattern, uint32_t n_guides, const char* const* guides,
                           const uint8_t* max_mm, cof_plan** out) {
    if (!out) return set_error(COF_E_ARG, "cof_plan_create: out is NULL");
    *out = nullptr;
    if (!pattern || !guides || !max_mm) return set_error(COF_E_ARG, "cof_plan_create: NULL argument");
    size_t L = strlen(pattern);
    if (L < 1 || L > COF_MAX_L) return set_error(COF_E_ARG, "pattern length %zu not in [1, %d]", L, COF_MAX_L);
    if (n_guides == 0 || n_guides > (1u << 24))
        return set_error(COF_E_ARG, "n_guides %u not in [1, 2^24]", n_guides);
    cof_plan* p = new cof_plan();
    p->L = (uint32_t)L;
    p->n_guides = n_guides;
    uint8_t pm[COF_MAX_L];
    for (size_t j = 0; j < L; j++) {
        pm[j] = iupac_mask(pattern[j]);
        if (!pm[j]) { delete p; return set_error(COF_E_ARG, "pattern[%zu]='%c' is not an IUPAC code", j, pattern[j]); }
        p->pattern.push_back((char)(pattern[j] >= 'a' ? pattern[j] - 32 : pattern[j]));
    }
    p->gmask.resize((size_t)n_guides * L);
    p->max_mm.assign(max_mm, max_mm + n_guides);
    for (uint32_t i = 0; i < n_guides; i++) {
        if (!guides[i]) { delete p; return set_error(COF_E_ARG, "guide %u is NULL", i); }
        if (max_mm[i] > L) {   // max_mm <= L (a larger threshold means the same: every PAM site)
            delete p;
            return set_error(COF_E_ARG, "guide %u: max_mm %u exceeds the pattern length %zu", i, (unsigned)max_mm[i], L);
        }
        if (strlen(guides[i]) != L) {
            delete p;
            return set_error(COF_E_ARG, "guide %u has length %zu, pattern has %zu", i, strlen(guides[i]), L);
        }
        std::string g;
        for (size_t j = 0; j < L; j++) {
            uint8_t m = iupac_mask(guides[i][j]);
            if (!m) { delete p; return set_error(COF_E_ARG, "guide %u[%zu]='%c' is not an IUPAC code", i, j, guides[i][j]); }
            p->gmask[(size_t)i * L + j] = m;
            g.push_back((char)(guides[i][j] >= 'a' ? guides[i][j] - 32 : guides[i][j]));
        }
        // the table comparer's 6-bit sums hold counts <= 63 (a 64-letter guide has no PAM)
        if (std::count(g.begin(), g.end(), 'N') == 0 && L == 64) {
            delete p;
            return set_error(COF_E_ARG, "guide %u compares all 64 positions (at most 63 supported)", i);
        }
        p->guides.push_back(g);
    }

    // ---- finder: non-N positions of the pattern ('+') and of its reverse complement ('-')
    for (int s = 0; s < 2; s++) {
        PamStrand& ps = p->pam[s];
        ps.n = 0;
        for (uint32_t j = 0; j < L; j++) {
            uint8_t m = s == 0 ? pm[j] : comp_mask(pm[L - 1 - j]);
            if (m != 15) { ps.j[ps.n] = (uint8_t)j; ps.set[ps.n] = m; ps.n++; }
        }
    }

    // guide letter mask in strand orientation (window offset j)
    auto gm = [&](int s, uint32_t i, uint32_t j) -> uint8_t {
        return s == 0 ? p->gmask[(size_t)i * L + j] : comp_mask(p->gmask[(size_t)i * L + (L - 1 - j)]);
    };

    // ---- host decoration: one-hot membership masks per guide and strand (window offsets)
    p->onehot.assign((size_t)2 * n_guides * 5, 0ull);
    for (int s = 0; s < 2; s++)
        for (uint32_t i = 0; i < n_guides; i++) {
            uint64_t* oh = &p->onehot[((size_t)s * n_guides + i) * 5];
            for (uint32_t j = 0; j < L; j++) {
                const uint8_t m = gm(s, i, j);
                for (int b = 0; b < 4; b++) oh[b] |= (uint64_t)((m >> b) & 1u) << j;
                if (m != 15) oh[4] |= 1ull << j;
            }
        }

    // ---- v1 comparer: group guides by (care mask, kind); records per strand
    // (32-bit care masks: built for L <= 32 only; longer patterns run the table comparer)
    std::map<std::pair<uint32_t, uint32_t>, std::vector<uint32_t>> groups;  // (care_fwd, kind) -> guides
    for (uint32_t i = 0; i < n_guides && L <= 32; i++) {
        uint32_t care = 0, kind = GROUP_CONCRETE;
        for (uint32_t j = 0; j < L; j++) {
            uint8_t m = gm(0, i, j);
            if (m != 15) care |= 1u << j;
            if (m != 15 && concrete_code(m) < 0) kind = GROUP_DEGENERATE;
        }
        if (kind == GROUP_DEGENERATE) p->any_degenerate = true;
        groups[{care, kind}].push_back(i);
    }
    std::vector<GroupDesc> gd[2];
    std::vector<uint32_t> recs[2];   // flattened uint4 records (4 words each)
    for (auto& kv : groups) {
        uint32_t kind = kv.first.second;
        for (int s = 0; s < 2; s++) {
            GroupDesc d;
            d.kind = kind;
            d.rec_begin = (uint32_t)(recs[s].size() / 4);
            d.n_guides = (uint32_t)kv.second.size();
            d.care = 0;
            for (uint32_t i : kv.second) {
                uint32_t lo = 0, hi = 0, care = 0, oh[4] = {0, 0, 0, 0};
                for (uint32_t j = 0; j < L; j++) {
                    uint8_t m = gm(s, i, j);
                    if (m == 15) continue;
                    care |= 1u << j;
                    for (int b = 0; b < 4; b++) if (m >> b & 1) oh[b] |= 1u << j;
                    int c = concrete_code(m);
                    if (c >= 0) { lo |= (uint32_t)(c & 1) << j; hi |= (uint32_t)(c >> 1) << j; }
                }
                d.care = care;
                uint32_t nt = (uint32_t)(-(int32_t)(p->max_mm[i] + 1));
                if (kind == GROUP_CONCRETE) {
                    recs[s].insert(recs[s].end(), {lo, hi, nt, i});
                } else {
                    recs[s].insert(recs[s].end(), {oh[0], oh[1], oh[2], oh[3]});
                    recs[s].insert(recs[s].end(), {care, nt, i, 0u});
                }
            }
            gd[s].push_back(d);
        }
    }
    p->n_groups = (uint32_t)gd[0].size();
    p->n_recs = (uint32_t)(recs[0].size() / 4);

    // ---- v2 comparer: bit-sliced pair tables over the union of compared positions
    p->n_blocks = (n_guides + 31) / 32;
    for (int s = 0; s < 2; s++) {
        uint64_t uc = 0;
        for (uint32_t i = 0; i < n_guides; i++)
            for (uint32_t j = 0; j < L; j++) if (gm(s, i, j) != 15) uc |= 1ull << j;
        p->union_care[s] = uc;
        PairLayout& pl = p->pairs[s];
        pl.n_pairs = 0;
        int pend = -1;
        for (uint32_t j = 0; j < L; j++) {
            if (!(uc >> j & 1)) continue;
            if (pend < 0) { pend = (int)j; continue; }
            pl.j1[pl.n_pairs] = (uint8_t)pend; pl.j2[pl.n_pairs] = (uint8_t)j; pl.n_pairs++;
            pend = -1;
        }
        if (pend >= 0) { pl.j1[pl.n_pairs] = (uint8_t)pend; pl.j2[pl.n_pairs] = 0xFF; pl.n_pairs++; }
        if (pl.n_pairs == 0) {   // all guides all-N: one dummy pair that never counts
            pl.j1[0] = 0; pl.j2[0] = 0xFF; pl.n_pairs = 1;
        }
        pl.n_real = pl.n_pairs;
        pl.n_cmp = (uint32_t)__builtin_popcountll(uc);
        pl.p0 = uc ? (uint32_t)__builtin_ctzll(uc) : 0u;
        const uint32_t span = uc ? 64u - (uint32_t)__builtin_clzll(uc) - pl.p0 : 1u;
        // two-word windows when the compared span exceeds one 32-bit word;
        // the wide kernels exist for multiples of 4 pairs: pad with pairs whose table
        // entries are all zero (they add nothing to any count)
        pl.wide = span > 32 ? 1u : 0u;
        if (pl.wide)
            while (pl.n_pairs % 4) { pl.j1[pl.n_pairs] = (uint8_t)pl.p0; pl.j2[pl.n_pairs] = 0xFE; pl.n_pairs++; }
        pl.contig = uc != 0 && (uc >> pl.p0) == (pl.n_cmp >= 64 ? ~0ull : ((1ull << pl.n_cmp) - 1ull)) &&
                    (pl.wide ? 2 * pl.n_pairs <= 64 : pl.p0 + 2 * pl.n_pairs <= 32);
    }
    // (both strands have the same number of compared positions, hence of pairs)
    const uint32_t NPAIR = p->pairs[0].n_pairs;
    if (p->pairs[1].n_pairs != NPAIR) { delete p; return set_error(COF_E_STATE, "internal: pair count mismatch"); }

    // ---- device image layout
    DevLayout& lay = p->lay;
    size_t off = 0;
    lay.counters = off; off = align256(off + 8 * sizeof(uint64_t));
    lay.groups_fwd = off; off = align256(off + gd[0].size() * sizeof(GroupDesc));
    lay.groups_rev = off; off = align256(off + gd[1].size() * sizeof(GroupDesc));
    lay.recs_fwd = off; off = align256(off + recs[0].size() * 4);
    lay.recs_rev = off; off = align256(off + recs[1].size() * 4);
    size_t ptab_bytes = (size_t)p->n_blocks * NPAIR * 25 * 8;
    lay.ptab_fwd = off; off = align256(off + ptab_bytes);
    lay.ptab_rev = off; off = align256(off + ptab_bytes);
    size_t pmeta_bytes = (size_t)p->n_blocks * 8 * 4;
    lay.pmeta_fwd = off; off = align256(off + pmeta_bytes);
    lay.pmeta_rev = off; off = align256(off + pmeta_bytes);
    lay.onehot = off; off = align256(off + p->onehot.size() * 8);
    // (rounded up to whole groups of 4 blocks: the single-pass kernel reads blocks four at a time)
    const size_t ftab_bytes = (size_t)((p->n_blocks + 3) & ~3u) * filter_block_words(NPAIR) * 4;
    lay.ftab_fwd = off; off = align256(off + ftab_bytes);
    lay.ftab_rev = off; off = align256(off + ftab_bytes);
    const size_t vrec_bytes = (size_t)((p->n_blocks + 3) & ~3u) * 32 * 2 * 16;
    lay.vrec_fwd = off; off = align256(off + vrec_bytes);
    lay.vrec_rev = off; off = align256(off + vrec_bytes);
    lay.total = off;
    p->image.assign(lay.total, 0);
    uint8_t* img = p->image.data();
    memcpy(img + lay.onehot, p->onehot.data(), p->onehot.size() * 8);
    memcpy(img + lay.groups_fwd, gd[0].data(), gd[0].size() * sizeof(GroupDesc));
    memcpy(img + lay.groups_rev, gd[1].data(), gd[1].size() * sizeof(GroupDesc));
    memcpy(img + lay.recs_fwd, recs[0].data(), recs[0].size() * 4);
    memcpy(img + lay.recs_rev, recs[1].data(), recs[1].size() * 4);
    for (int s = 0; s < 2; s++) {
        uint32_t* tab = (uint32_t*)(img + (s == 0 ? lay.ptab_fwd : lay.ptab_rev));
        uint32_t* meta = (uint32_t*)(img + (s == 0 ? lay.pmeta_fwd : lay.pmeta_rev));
        const PairLayout& pl = p->pairs[s];
        for (uint32_t b = 0; b < p->n_blocks; b++) {
            uint32_t valid = 0, T[6] = {0, 0, 0, 0, 0, 0};
            for (uint32_t k = 0; k < 32; k++) {
                uint32_t i = b * 32 + k;
                if (i >= n_guides) break;
                valid |= 1u << k;
                uint32_t t = p->max_mm[i] > 63 ? 63 : p->max_mm[i];
                for (int w = 0; w < 6; w++) T[w] |= ((t >> w) & 1u) << k;
            }
            for (int w = 0; w < 6; w++) meta[b * 8 + w] = T[w];
            meta[b * 8 + 6] = valid;
            for (uint32_t q = 0; q < NPAIR; q++) {
                for (uint32_t c = 0; c < 25; c++) {
                    uint32_t b1 = c / 5, b2 = c % 5;   // 0..3 = A,C,G,T ; 4 = N
                    uint32_t w0 = 0, w1 = 0;
                    for (uint32_t k = 0; k < 32; k++) {
                        uint32_t i = b * 32 + k;
                        if (i >= n_guides) break;
                        auto mis = [&](uint32_t j, uint32_t base) -> uint32_t {
                            uint8_t m = gm(s, i, j);
                            if (m == 15) return 0;                  // not compared
                            if (base == 4) return 1;                // genome N: always a mismatch (G2)
                            return (m >> base & 1) ? 0 : 1;
                        };
                        if (q >= pl.n_real) break;             // padding pair: all zero
                        uint32_t cnt = mis(pl.j1[q], b1);
                        if (pl.j2[q] != 0xFF) cnt += mis(pl.j2[q], b2);
                        if (pl.j2[q] == 0xFF && p->union_care[s] == 0) cnt = 0;
                        w0 |= (cnt & 1u) << k;
                        w1 |= (cnt >> 1) << k;
                    }
                    size_t e = (size_t)b * NPAIR * 25 + pair_entry(NPAIR, q, b1, b2);
                    tab[e * 2 + 0] = w0;
                    tab[e * 2 + 1] = w1;
                    // single-pass filter: the pair has at least one mismatch (count 1 or 2);
                    // guides past the plan always "mismatch" (ACGT entries only)
                    if (b1 < 4 && b2 < 4) {
                        uint32_t* ft = (uint32_t*)(img + (s == 0 ? lay.ftab_fwd : lay.ftab_rev));
                        const uint32_t nv = n_guides - b * 32 >= 32 ? 0u : ~0u << (n_guides - b * 32);
                        ft[(size_t)b * filter_block_words(NPAIR) + pair_entry(NPAIR, q, b1, b2)] = w0 | w1 | nv;
                    }
                }
            }
        }
        {   // padding blocks of the last group of 4: no guide, every bit set
            uint32_t* ft = (uint32_t*)(img + (s == 0 ? lay.ftab_fwd : lay.ftab_rev));
            for (uint32_t b = p->n_blocks; b < ((p->n_blocks + 3) & ~3u); b++)
                for (uint32_t w = 0; w < filter_block_words(NPAIR); w++) ft[(size_t)b * filter_block_words(NPAIR) + w] = ~0u;
        }
        // single-pass verification records, window offsets relative to p0 (compared spans
        // <= 32 only): {lo, hi, care, t} of the concrete letters and the one-hot {A, C, G, T}
        // membership of every letter
        if (!pl.wide) {
            uint32_t* vr = (uint32_t*)(img + (s == 0 ? lay.vrec_fwd : lay.vrec_rev));
            for (uint32_t i = 0; i < n_guides; i++) {
                uint32_t lo = 0, hi = 0, care = 0, oh[4] = {0, 0, 0, 0};
                for (uint32_t j = pl.p0; j < L && j < pl.p0 + 32; j++) {
                    const uint8_t m = gm(s, i, j);
                    if (m == 15) continue;
                    const uint32_t bit = 1u << (j - pl.p0);
                    care |= bit;
                    for (int bb = 0; bb < 4; bb++) if (m >> bb & 1) oh[bb] |= bit;
                    const int c = concrete_code(m);
                    if (c >= 0) { lo |= (c & 1) ? bit : 0u; hi |= (c >> 1) ? bit : 0u; }
                }
                uint32_t* r = vr + (size_t)i * 8;
                r[0] = lo; r[1] = hi; r[2] = care; r[3] = p->max_mm[i];
                r[4] = oh[0]; r[5] = oh[1]; r[6] = oh[2]; r[7] = oh[3];
            }
        }
    }
    *out = p;
    return COF_OK;
}

void cof_plan_destroy(cof_plan* p) { delete p; }
uint32_t cof_plan_length(const cof_plan* p) { return p ? p->L : 0; }
uint32_t cof_plan_n_guides(const cof_plan* p) { return p ? p->n_guides : 0; }
size_t cof_plan_device_bytes(const cof_plan* p) { return p ? p->lay.total : 0; }

cof_status cof_plan_upload(const cof_plan* p, void* plan_dev, cof_stream s) {
    if (!p || !plan_dev) return set_error(COF_E_ARG, "cof_plan_upload: NULL argument");
    if ((uintptr_t)plan_dev & 255) return set_error(COF_E_ARG, "cof_plan_upload: plan_dev not 256-byte aligned");
    cudaError_t e = cudaMemcpyAsync(plan_dev, p->image.data(), p->image.size(), cudaMemcpyHostToDevice,
                                    (cudaStream_t)s);
    if (e != cudaSuccess) return cuda_error(e, "cof_plan_upload");
    return COF_OK;
}

}  // extern "C"
