"""The single-pass comparer's filter circuits (csrc/filter_circuit.cuh: generated
carry-save counts nz_count<NP> and the hand-reduced count-vs-threshold circuits of the
configs' shapes) checked EXHAUSTIVELY on the host: for every assignment of the NP one-bit
inputs (bit-sliced 32 per word, like the kernel) the surviving guides must be exactly
those whose number of set inputs is <= the threshold, for uniform thresholds (the
specialised and the generic borrow-chain comparators) and per-guide threshold planes.
The circuit is the product's code compiled by g++; the expected value is a popcount."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_socc_jinv23_b200", "csrc")

SRC = r'''
#include <cstdio>
#include <cstdint>
#define __device__
#define __forceinline__ inline
#define COF_FC inline
#include "filter_circuit.cuh"
using namespace cof;

template <int NP, int TC>
static long check() {
    long bad = 0;
    const uint32_t n = 1u << NP;
    for (uint32_t x0 = 0; x0 < n; x0 += 32) {
        uint32_t v[NP];
        for (int q = 0; q < NP; q++) {
            v[q] = 0;
            for (int j = 0; j < 32; j++) v[q] |= ((((x0 + j) >> q) & 1u)) << j;
        }
        // uniform threshold TC (specialised circuit where one exists, else the borrow chain)
        uint32_t meta[8] = {0, 0, 0, 0, 0, 0, 0xFFFFFFFFu, 0};
        const uint32_t pass = filter_pass<NP, TC>(v, meta);
        // per-guide thresholds (generic borrow chain): lane j gets threshold (j * 7 + TC) % (NP + 2)
        uint32_t tpl[8] = {0, 0, 0, 0, 0, 0, 0xFFFFFFFFu, 0};
        for (int j = 0; j < 32; j++) {
            const uint32_t t = (uint32_t)(j * 7 + TC) % (NP + 2);
            for (int w = 0; w < 6; w++) tpl[w] |= ((t >> w) & 1u) << j;
        }
        const uint32_t pass_g = filter_pass<NP, -1>(v, tpl);
        for (int j = 0; j < 32; j++) {
            const int cnt = __builtin_popcount((x0 + j) & (n - 1));
            const uint32_t tg = (uint32_t)(j * 7 + TC) % (NP + 2);
            bad += (((pass >> j) & 1u) != (cnt <= TC ? 1u : 0u));
            bad += (((pass_g >> j) & 1u) != ((uint32_t)cnt <= tg ? 1u : 0u));
        }
    }
    return bad;
}

#define CHECK(NP, TC) do { long b = check<NP, TC>(); printf("NP=%d TC=%d bad=%ld\n", NP, TC, b); bad += b; } while (0)

int main() {
    long bad = 0;
    CHECK(10, 4); CHECK(10, 5); CHECK(10, 6);     // hand-reduced
    CHECK(12, 5);                                  // hand-reduced
    CHECK(1, 0); CHECK(3, 1); CHECK(7, 2); CHECK(10, 3); CHECK(11, 4); CHECK(12, 6); CHECK(13, 7);
    CHECK(15, 5); CHECK(16, 7); CHECK(16, 15); CHECK(9, 0);
    return bad ? 1 : 0;
}
'''


def test_filter_circuits_exhaustive(tmp_path):
    src = tmp_path / "fc.cpp"
    src.write_text(SRC)
    exe = tmp_path / "fc"
    subprocess.run(["g++", "-O2", "-std=c++17", "-I", CSRC, str(src), "-o", str(exe)], check=True)
    r = subprocess.run([str(exe)], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout
    assert r.stdout.count("bad=0") == 15
