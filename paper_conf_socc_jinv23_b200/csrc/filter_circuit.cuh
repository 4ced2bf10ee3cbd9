// Filter circuits of the single-pass comparer (single.cu): from the NP one-bit inputs
// v[q] (bit k = guide k's position pair q holds >= 1 mismatch) to the guides that
// survive, i.e. whose number of mismatched pairs is <= their threshold.  Plain bit
// operations (each line lowers to LOP3s), usable on the host so that
// tests/test_filter_circuit.py can check them exhaustively against popcounts.
#pragma once
#include <cstdint>
#include "csa_gen.cuh"

#ifndef COF_FC
#define COF_FC __device__ __forceinline__
#endif

namespace cof {

COF_FC uint32_t maj3(uint32_t x, uint32_t y, uint32_t z) { return (x & y) | (x & z) | (y & z); }

// Hand-reduced filter circuits for the configs' shapes: the carry-save count of NP one-bit
// inputs fused with the constant-threshold comparison (each line one LOP3).  "fail" =
// the number of mismatched pairs exceeds TC.  Derivation (NP = 10): three full adders over
// v0..v8 (sums s1..s3, carries c1..c3) and FA(s1, s2, s3) = (S, C) give S (weight 1) and
// C, c1..c3 (weight 2); FA(c1, c2, c3) = (e, f);
// with x0 = S ^ v9 (count bit 0) and k0 = S & v9, the weight-2 column is (e, C, k0):
// bit1 = XOR3, f2 = MAJ; the weight-4 column (f, f2) gives bit2 = f ^ f2, bit3 = f & f2.
//   count >= 7  <=>  bit3 | bit2 & bit1 & bit0  =  MAJ(f, f2, bit1 & bit0), and
//                    bit1 & bit0 = (e ^ C) & x0   (x0 = 1 forces k0 = 0)
//   count >= 6  <=>  MAJ(f, f2, bit1);   count >= 5  <=>  MAJ(f, f2, bit1 | bit0)
// NP = 12, TC = 5: count = bit0 + 2 rest with rest = c1 + c2 + c3 + c4 + C + k0 (four full
// adders over v0..v11, FA(s1, s2, s3) = (S, C), k0 = S & s4), and count >= 6 <=> rest >= 3
// <=> MAJ(f1, f2, e1 | e2) with (e1, f1) = FA(c1, c2, c3), (e2, f2) = FA(c4, C, k0).
// Returns false (no specialisation) through `done`.
template <int NP, int TC>
COF_FC uint32_t filter_fail_fast(const uint32_t (&v)[NP], bool& done) {
    done = false;
    if constexpr (NP == 10 && (TC == 4 || TC == 5 || TC == 6)) {
        const uint32_t s1 = v[0] ^ v[1] ^ v[2], c1 = maj3(v[0], v[1], v[2]);
        const uint32_t s2 = v[3] ^ v[4] ^ v[5], c2 = maj3(v[3], v[4], v[5]);
        const uint32_t s3 = v[6] ^ v[7] ^ v[8], c3 = maj3(v[6], v[7], v[8]);
        const uint32_t S = s1 ^ s2 ^ s3, C = maj3(s1, s2, s3);
        const uint32_t e = c1 ^ c2 ^ c3, f = maj3(c1, c2, c3);
        const uint32_t k0 = S & v[9];
        const uint32_t f2 = maj3(e, C, k0);
        done = true;
        if constexpr (TC == 6) return maj3(f, f2, (e ^ C) & (S ^ v[9]));
        else if constexpr (TC == 5) return maj3(f, f2, e ^ C ^ k0);
        else return maj3(f, f2, (e ^ C ^ k0) | (S ^ v[9]));
    } else if constexpr (NP == 12 && TC == 5) {
        const uint32_t s1 = v[0] ^ v[1] ^ v[2], c1 = maj3(v[0], v[1], v[2]);
        const uint32_t s2 = v[3] ^ v[4] ^ v[5], c2 = maj3(v[3], v[4], v[5]);
        const uint32_t s3 = v[6] ^ v[7] ^ v[8], c3 = maj3(v[6], v[7], v[8]);
        const uint32_t s4 = v[9] ^ v[10] ^ v[11], c4 = maj3(v[9], v[10], v[11]);
        const uint32_t S = s1 ^ s2 ^ s3, C = maj3(s1, s2, s3);
        const uint32_t k0 = S & s4;
        const uint32_t e1 = c1 ^ c2 ^ c3, f1 = maj3(c1, c2, c3);
        const uint32_t e2 = c4 ^ C ^ k0, f2 = maj3(c4, C, k0);
        done = true;
        return maj3(f1, f2, e1 | e2);
    }
    return 0u;
}

// Filter: bit k of the result = guide k of the block survives (its number of pairs with a
// mismatch is <= its threshold).  TC >= 0: one threshold for every guide of the launch,
// TC < NP; guides past the plan need no mask there, their table bits are all set (count
// NP > TC).  TC < 0: per-guide threshold planes m[0..5] and the valid-guide mask m[6].
template <int NP, int TC>
COF_FC uint32_t filter_pass(const uint32_t (&v)[NP], const uint32_t* __restrict__ m) {
    static_assert(TC < NP, "a uniform threshold below the pair count");
    bool fast;
    const uint32_t ff = filter_fail_fast<NP, TC>(v, fast);
    if (fast) return ~ff;
    uint32_t c[5];
    nz_count<NP>(v, c);
    uint32_t bw;                       // borrow out of (t - count): set where count > t
    if constexpr (TC >= 0) {
        bw = (TC & 1) ? 0u : c[0];
#pragma unroll
        for (int w = 1; w < 5; w++) bw = ((TC >> w) & 1) ? (c[w] & bw) : (c[w] | bw);
        return ~bw;
    } else {
        bw = c[0] & ~m[0];
#pragma unroll
        for (int w = 1; w < 6; w++) {
            const uint32_t cw = w < 5 ? c[w] : 0u;
            bw = (~m[w] & cw) | (~m[w] & bw) | (cw & bw);
        }
    }
    return m[6] & ~bw;
}

}  // namespace cof
