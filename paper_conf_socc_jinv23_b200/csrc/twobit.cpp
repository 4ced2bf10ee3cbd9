// UCSC .2bit genome reader (the genome formats users hold; the paper's
// host "reads genome sequence data in single- or multi-sequence data format").
//
// A .2bit file packs 4 bases per byte (first base in the top two bits; T=0 C=1 A=2 G=3),
// lists N runs as (start, size) blocks and soft-mask runs as mask blocks.  Packing into
// the product's planes (A=00 C=01 G=10 T=11, lo = bit 0; nm = 1 for N) is a per-byte table
// lookup: for 2bit code v = (b1 b0), lo = !b1 and hi = !(b1 ^ b0).  Mask blocks are
// ignored (case-insensitive, reading G4); N blocks set nm and clear lo/hi (G2).
#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include "cof_internal.h"

using namespace cof;

struct cof_twobit {
    int fd = -1;
    const uint8_t* data = nullptr;
    size_t size = 0;
    bool swap = false;
    struct Rec {
        std::string name;
        uint64_t length = 0;
        size_t dna_off = 0;                   // first packed byte
        std::vector<uint32_t> nstart, nsize;  // N blocks, ascending
    };
    std::vector<Rec> recs;
};

namespace {

struct Lut {
    uint8_t lo[256], hi[256];   // 4 bases of a byte: bit j = base j (j = 0 is the top pair)
    Lut() {
        for (int b = 0; b < 256; b++) {
            uint8_t l = 0, h = 0;
            for (int j = 0; j < 4; j++) {
                const int v = (b >> (6 - 2 * j)) & 3;
                const int b1 = v >> 1, b0 = v & 1;
                l |= (uint8_t)((b1 ^ 1) << j);
                h |= (uint8_t)(((b1 ^ b0) ^ 1) << j);
            }
            lo[b] = l;
            hi[b] = h;
        }
    }
} g_lut;

bool rd32(const cof_twobit* t, size_t off, uint32_t& v) {
    if (off + 4 > t->size) return false;
    uint32_t x;
    memcpy(&x, t->data + off, 4);
    v = t->swap ? __builtin_bswap32(x) : x;
    return true;
}

bool rd64(const cof_twobit* t, size_t off, uint64_t& v) {
    if (off + 8 > t->size) return false;
    uint64_t x;
    memcpy(&x, t->data + off, 8);
    v = t->swap ? __builtin_bswap64(x) : x;
    return true;
}

}  // namespace

extern "C" {

cof_status cof_2bit_open(const char* path, cof_twobit** out) {
    if (!path || !out) return set_error(COF_E_ARG, "cof_2bit_open: NULL argument");
    *out = nullptr;
    int fd = open(path, O_RDONLY);
    if (fd < 0) return set_error(COF_E_IO, "cannot open %s", path);
    struct stat st;
    if (fstat(fd, &st) != 0) { close(fd); return set_error(COF_E_IO, "cannot stat %s", path); }
    cof_twobit* t = new cof_twobit();
    t->fd = fd;
    t->size = (size_t)st.st_size;
    if (t->size) {
        void* m = mmap(nullptr, t->size, PROT_READ, MAP_PRIVATE, fd, 0);
        if (m == MAP_FAILED) { close(fd); delete t; return set_error(COF_E_IO, "cannot mmap %s", path); }
        t->data = (const uint8_t*)m;
    }
    auto fail = [&](const char* what) {
        cof_2bit_close(t);
        return set_error(COF_E_IO, "%s: %s", path, what);
    };
    uint32_t sig = 0, version = 0, count = 0;
    if (!rd32(t, 0, sig)) return fail("truncated header");
    if (sig == 0x4327411Au) t->swap = true;
    else if (sig != 0x1A412743u) return fail("not a .2bit file (bad signature)");
    if (!rd32(t, 4, version) || !rd32(t, 8, count)) return fail("truncated header");
    if (version > 1) return fail("unsupported .2bit version");
    size_t off = 16;
    for (uint32_t k = 0; k < count; k++) {
        if (off >= t->size) return fail("truncated index");
        const uint32_t nl = t->data[off++];
        if (off + nl > t->size) return fail("truncated index");
        cof_twobit::Rec r;
        r.name.assign((const char*)t->data + off, nl);
        off += nl;
        uint64_t roff = 0;
        if (version == 0) {
            uint32_t o32;
            if (!rd32(t, off, o32)) return fail("truncated index");
            roff = o32;
            off += 4;
        } else {
            if (!rd64(t, off, roff)) return fail("truncated index");
            off += 8;
        }
        uint32_t dna = 0, nb = 0, mb = 0;
        size_t p = (size_t)roff;
        if (!rd32(t, p, dna) || !rd32(t, p + 4, nb)) return fail("truncated record header");
        p += 8;
        r.nstart.resize(nb);
        r.nsize.resize(nb);
        for (uint32_t b = 0; b < nb; b++)
            if (!rd32(t, p + 4ull * b, r.nstart[b])) return fail("truncated N blocks");
        p += 4ull * nb;
        for (uint32_t b = 0; b < nb; b++)
            if (!rd32(t, p + 4ull * b, r.nsize[b])) return fail("truncated N blocks");
        p += 4ull * nb;
        if (!rd32(t, p, mb)) return fail("truncated mask blocks");
        p += 4 + 8ull * mb + 4;   // mask starts + sizes + reserved word
        r.length = dna;
        r.dna_off = p;
        if (p + (dna + 3ull) / 4 > t->size) return fail("truncated sequence data");
        for (uint32_t b = 0; b < nb; b++)
            if ((uint64_t)r.nstart[b] + r.nsize[b] > dna) return fail("N block past the sequence end");
        t->recs.push_back(std::move(r));
    }
    *out = t;
    return COF_OK;
}

void cof_2bit_close(cof_twobit* t) {
    if (!t) return;
    if (t->data) munmap((void*)t->data, t->size);
    if (t->fd >= 0) close(t->fd);
    delete t;
}

uint32_t cof_2bit_count(const cof_twobit* t) { return t ? (uint32_t)t->recs.size() : 0; }
const char* cof_2bit_name(const cof_twobit* t, uint32_t i) {
    return (t && i < t->recs.size()) ? t->recs[i].name.c_str() : nullptr;
}
uint64_t cof_2bit_length(const cof_twobit* t, uint32_t i) {
    return (t && i < t->recs.size()) ? t->recs[i].length : 0;
}

cof_status cof_2bit_pack(const cof_twobit* t, uint32_t i, uint64_t first, uint64_t n, uint32_t* lo, uint32_t* hi,
                         uint32_t* nm) {
    if (!t || !lo || !hi || !nm) return set_error(COF_E_ARG, "cof_2bit_pack: NULL argument");
    if (i >= t->recs.size()) return set_error(COF_E_ARG, "cof_2bit_pack: record %u out of range", i);
    const auto& r = t->recs[i];
    if (first + n > r.length) return set_error(COF_E_ARG, "cof_2bit_pack: range past record end");
    const uint8_t* dna = t->data + r.dna_off;
    const uint64_t nbytes = (r.length + 3) / 4;
    const uint64_t words = cof_plane_words(n);
    const int64_t used = (int64_t)((n + 31) / 32);
#pragma omp parallel for schedule(static) if (n > (1u << 20))
    for (int64_t w = 0; w < used; w++) {
        const uint64_t s = first + 32ull * (uint64_t)w;       // first base of the word
        const uint64_t b0 = s >> 2;
        const int rsh = (int)(s & 3);
        uint64_t l36 = 0, h36 = 0;                             // bases from 4 * b0 on
        for (int b = 0; b < 9; b++) {
            if (b0 + b >= nbytes) break;
            const uint8_t byte = dna[b0 + b];
            l36 |= (uint64_t)g_lut.lo[byte] << (4 * b);
            h36 |= (uint64_t)g_lut.hi[byte] << (4 * b);
        }
        const uint64_t cnt = std::min<uint64_t>(32, n - 32ull * (uint64_t)w);
        const uint32_t valid = cnt >= 32 ? 0xFFFFFFFFu : ((1u << cnt) - 1u);
        lo[w] = (uint32_t)(l36 >> rsh) & valid;
        hi[w] = (uint32_t)(h36 >> rsh) & valid;
        nm[w] = ~valid;
    }
    for (uint64_t w = (uint64_t)used; w < words; w++) { lo[w] = 0; hi[w] = 0; nm[w] = ~0u; }
    // N blocks overlapping [first, first + n)
    auto it = std::upper_bound(r.nstart.begin(), r.nstart.end(), (uint32_t)std::min<uint64_t>(first, 0xFFFFFFFFu));
    size_t b = it == r.nstart.begin() ? 0 : (size_t)(it - r.nstart.begin()) - 1;
    for (; b < r.nstart.size(); b++) {
        const uint64_t a = r.nstart[b], e = a + r.nsize[b];
        if (a >= first + n) break;
        if (e <= first) continue;
        uint64_t x = std::max(a, first) - first, y = std::min(e, first + n) - first;
        while (x < y) {
            const uint64_t w = x >> 5;
            const uint32_t bit = (uint32_t)(x & 31);
            const uint32_t take = (uint32_t)std::min<uint64_t>(32 - bit, y - x);
            const uint32_t m = (take >= 32 ? 0xFFFFFFFFu : ((1u << take) - 1u)) << bit;
            nm[w] |= m;
            lo[w] &= ~m;
            hi[w] &= ~m;
            x += take;
        }
    }
    return COF_OK;
}

}  // extern "C"
