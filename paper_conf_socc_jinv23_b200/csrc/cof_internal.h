// Internal definitions shared by the libcof.so translation units (NOT by the oracle).
#pragma once
#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>

#include "../../include/cof.h"

namespace cof {

// ---- error handling (thread-local message, COF_* status codes)
cof_status set_error(cof_status code, const char* fmt, ...);
cof_status cuda_error(int err, const char* what);   // err = cudaError_t
void count_launches(uint64_t n);

// ---- nucleotide encoding of the product path
// 4-bit IUPAC set masks: A=1, C=2, G=4, T=8 (N = 15).  Returns 0 for a non-IUPAC letter.
uint8_t iupac_mask(char c);
inline uint8_t comp_mask(uint8_t m) {          // complement of a set: A<->T, C<->G
    return (uint8_t)(((m & 1) << 3) | ((m & 8) >> 3) | ((m & 2) << 1) | ((m & 4) >> 1));
}
// 2-bit code of a concrete base set (A=0 C=1 G=2 T=3), -1 if not a single base.
inline int concrete_code(uint8_t m) {
    switch (m) { case 1: return 0; case 2: return 1; case 4: return 2; case 8: return 3; default: return -1; }
}

// ---- finder parameters (per strand, non-N pattern positions)
struct PamStrand {
    uint32_t n;            // number of non-N positions
    uint8_t j[COF_MAX_L];      // window offset
    uint8_t set[COF_MAX_L];    // IUPAC set mask
};

// ---- comparer guide tables (device image inside plan_dev)
// Concrete group record (uint4): {lo, hi, (uint32)-(t+1), guide}
// Degenerate group record (2 x uint4): {A, C, G, T one-hot}, {care, -(t+1), guide, 0}
enum GroupKind : uint32_t { GROUP_CONCRETE = 0, GROUP_DEGENERATE = 1 };
struct GroupDesc {
    uint32_t care;         // compared-position mask (bit j = window offset j)
    uint32_t kind;
    uint32_t rec_begin;    // index into the strand's uint4 record array
    uint32_t n_guides;
};

#ifdef __CUDACC__
#define COF_HD __host__ __device__ __forceinline__
#else
#define COF_HD inline
#endif

// Entry of a base pair (b1, b2 in 0..3 = A,C,G,T, 4 = N) of pair q in a 32-guide block of
// the pair table (NP pairs, 25 entries each).  The 16 ACGT combos of a pair are 16
// consecutive 8-byte entries (128 bytes = every shared-memory bank exactly once, so a
// half-warp of lookups into one pair never conflicts); the 9 rare N combos of all pairs
// follow in a separate region.  Inside the 16 the index is lo(b1) | lo(b2)<<1 | hi(b1)<<2 |
// hi(b2)<<3 (lo/hi = the two bits of the 2-bit code): for two adjacent window positions
// that is one nibble of (lo-plane bits | hi-plane bits << 2), see the comparer's fast path.
COF_HD uint32_t pair_entry(uint32_t np, uint32_t q, uint32_t b1, uint32_t b2) {
    if (b1 < 4 && b2 < 4) return q * 16u + ((b1 & 1u) | ((b2 & 1u) << 1) | ((b1 >> 1) << 2) | ((b2 >> 1) << 3));
    return np * 16u + q * 9u + (b1 == 4 ? b2 : 5u + b1);
}

// Single-pass comparer filter table (single.cu): per strand and 32-guide block, per
// position pair, the 16 ACGT one-word entries (bit k = guide k's pair has >= 1 mismatch
// for that base pair), indexed like pair_entry's ACGT part: 64 bytes per pair, addressed by
// OR-ing the pair nibble in.  No N entries: the filter reads a genome N as the A its
// planes hold (lo = hi = 0), which can only hide mismatches, so the filter stays a
// necessary condition and the exact verification counts the N.  Guides past the plan
// (the last block's padding, padding blocks) have every bit set: they never survive.
COF_HD uint32_t filter_block_words(uint32_t np) { return np * 16u; }

// Bit-sliced pair-table comparer (v2): per strand, per 32-guide block, per position pair,
// 25 entries (base pair combos incl. N) of {bit0, bit1} mismatch-count planes.
struct PairLayout {
    uint32_t n_pairs;          // pairs covering the union of compared positions (+ padding)
    uint8_t j1[32], j2[32];    // window offsets of the pair (j2 == 0xFF: single position,
                               // 0xFE: padding pair, table entries all zero)
    uint32_t contig;           // 1: compared positions are the contiguous range [p0, p0 + n_cmp)
    uint32_t p0, n_cmp;        //    so pair q = window offsets (p0 + 2q, p0 + 2q + 1)
    uint32_t wide;             // 1: compared span > 32: 64-bit windows, n_pairs a multiple of 4
    uint32_t n_real;           // pairs before the padding
};

// Device plan image layout (byte offsets from plan_dev; all 256-byte aligned)
struct DevLayout {
    size_t counters;           // uint64[8]: n_fwd, n_rev, n_hits, ...
    size_t groups_fwd, groups_rev;   // GroupDesc[n_groups]
    size_t recs_fwd, recs_rev;       // uint4[n_recs]
    size_t ptab_fwd, ptab_rev;       // pair tables: uint2[n_blocks][n_pairs][25]
    size_t pmeta_fwd, pmeta_rev;     // per block: uint32[8] = {T0..T5 threshold planes, valid, 0}
    size_t onehot;                   // uint64[2][n_guides][5] decoration masks (see cof_plan::onehot)
    size_t ftab_fwd, ftab_rev;       // single-pass filter tables: uint32[n_blocks][filter_block_words(np)]
    size_t vrec_fwd, vrec_rev;       // single-pass verification records: uint4[n_blocks * 32][2]
    size_t total;
};

}  // namespace cof

struct cof_plan {
    uint32_t L = 0;
    uint32_t n_guides = 0;
    std::string pattern;                 // upper-case
    std::vector<std::string> guides;     // upper-case
    std::vector<uint8_t> max_mm;
    std::vector<uint8_t> gmask;          // [n_guides * L] IUPAC masks (forward orientation)
    std::vector<uint64_t> onehot;        // [2][n_guides][5]: A, C, G, T membership + care, window offsets
    cof::PamStrand pam[2];               // [0] '+', [1] '-' (reverse-complemented pattern)
    uint32_t n_groups = 0;
    uint32_t n_recs = 0;
    uint32_t n_blocks = 0;               // 32-guide blocks (pair-table comparer)
    cof::PairLayout pairs[2];
    uint64_t union_care[2] = {0, 0};
    bool any_degenerate = false;
    cof::DevLayout lay;
    std::vector<uint8_t> image;          // host copy of the device image (counters zeroed)
};
