// Host side of the boundary: errors, version, launch counter, the 2-bit packer (M4), the
// indexed FASTA reader (M2), chunk loading (M11), counters, collect (M10) and merge.
//
// Paper: P:L29 (host reads single/multi-sequence files, divides the genome into chunks,
// collects "chromosome number, position, direction, the number of mismatched bases and
// potential off-target DNA sequence with mismatched bases"); P:L289 ("2-bit sequence
// format", OpenMP in the host program).
#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <queue>
#include <string>
#include <vector>

#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <cuda_runtime.h>
#include <emmintrin.h>
#include <omp.h>

#include "cof_internal.h"

namespace cof {

static thread_local std::string g_err;
static std::atomic<uint64_t> g_launches{0};

cof_status set_error(cof_status code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

cof_status cuda_error(int err, const char* what) {
    return set_error(COF_E_CUDA, "%s: %s", what, cudaGetErrorString((cudaError_t)err));
}

void count_launches(uint64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

// byte -> 2-bit code (A0 C1 G2 T3) or 4 for anything else (N, IUPAC, junk): readings G2/G4
static uint8_t g_code[256];
static struct CodeInit {
    CodeInit() {
        for (int i = 0; i < 256; i++) g_code[i] = 4;
        g_code['A'] = g_code['a'] = 0;
        g_code['C'] = g_code['c'] = 1;
        g_code['G'] = g_code['g'] = 2;
        g_code['T'] = g_code['t'] = 3;
    }
} g_code_init;

// Pack 32 codes into one word of each plane.
static inline void pack_word(const uint8_t* codes, int n, uint32_t& lo, uint32_t& hi, uint32_t& nm) {
    uint32_t l = 0, h = 0, m = 0;
    for (int b = 0; b < n; b++) {
        uint32_t c = codes[b];
        l |= (uint32_t)(c & 1) << b;
        h |= (uint32_t)((c >> 1) & 1) << b;
        m |= (uint32_t)(c >> 2) << b;
    }
    l &= ~m; h &= ~m;                     // N: lo = hi = 0
    if (n < 32) m |= ~0u << n;            // past the end: N
    lo = l; hi = h; nm = m;
}

// Pack 32 ASCII bases (any case) into one word of each plane, SSE2 (baseline x86-64):
// clearing bit 5 folds exactly {X, x} onto X, so the four byte compares against A/C/G/T
// give the same codes as g_code; every other byte is N (lo = hi = 0).
static inline void pack32_ascii(const char* s, uint32_t& lo, uint32_t& hi, uint32_t& nm) {
    const __m128i fold = _mm_set1_epi8((char)0xDF);
    const __m128i a = _mm_and_si128(_mm_loadu_si128((const __m128i*)s), fold);
    const __m128i b = _mm_and_si128(_mm_loadu_si128((const __m128i*)(s + 16)), fold);
    auto eq = [&](char ch) -> uint32_t {
        const __m128i c = _mm_set1_epi8(ch);
        return (uint32_t)_mm_movemask_epi8(_mm_cmpeq_epi8(a, c)) |
               ((uint32_t)_mm_movemask_epi8(_mm_cmpeq_epi8(b, c)) << 16);
    };
    const uint32_t A = eq('A'), C = eq('C'), G = eq('G'), T = eq('T');
    lo = C | T;
    hi = G | T;
    nm = ~(A | C | G | T);
}

}  // namespace cof

using namespace cof;

extern "C" {

const char* cof_last_error(void) { return g_err.c_str(); }
const char* cof_version(void) { return "cof-b200 0.1 (sm_100a)"; }

int cof_set_host_threads(int n) {
    if (n > 0) omp_set_num_threads(n);
    return omp_get_max_threads();
}
uint64_t cof_launch_count(void) { return g_launches.load(); }

uint64_t cof_plane_words(uint64_t n_bases) {
    // ceil(n/32) data words, rounded up to a finder tile (512 words), + 4 pad words so the
    // finder's 16-byte-granular bulk copies of (tile + halo) never leave the allocation.
    uint64_t w = (n_bases + 31) / 32;
    return ((w + 511) / 512) * 512 + 4;
}

cof_status cof_pack(const char* ascii, uint64_t n, uint32_t* lo, uint32_t* hi, uint32_t* nm) {
    if ((!ascii && n) || !lo || !hi || !nm) return set_error(COF_E_ARG, "cof_pack: NULL argument");
    const uint64_t words = cof_plane_words(n);
    const int64_t full = (int64_t)(n / 32);
#pragma omp parallel for schedule(static)
    for (int64_t w = 0; w < full; w++) pack32_ascii(ascii + w * 32, lo[w], hi[w], nm[w]);
    uint64_t w = (uint64_t)full;
    if (n % 32) {
        uint8_t codes[32];
        int r = (int)(n % 32);
        for (int b = 0; b < r; b++) codes[b] = g_code[(uint8_t)ascii[w * 32 + b]];
        pack_word(codes, r, lo[w], hi[w], nm[w]);
        w++;
    }
    for (; w < words; w++) { lo[w] = 0; hi[w] = 0; nm[w] = ~0u; }
    return COF_OK;
}

cof_status cof_unpack(const uint32_t* lo, const uint32_t* hi, const uint32_t* nm, uint64_t first,
                      uint64_t n, char* ascii) {
    if (!lo || !hi || !nm || (!ascii && n)) return set_error(COF_E_ARG, "cof_unpack: NULL argument");
    static const char B[4] = {'A', 'C', 'G', 'T'};
#pragma omp parallel for schedule(static) if (n > (1u << 20))
    for (int64_t i = 0; i < (int64_t)n; i++) {
        uint64_t p = first + (uint64_t)i;
        uint64_t w = p >> 5;
        int b = (int)(p & 31);
        if (nm[w] >> b & 1) ascii[i] = 'N';
        else ascii[i] = B[((lo[w] >> b) & 1) | (((hi[w] >> b) & 1) << 1)];
    }
    return COF_OK;
}

cof_status cof_valid_starts(const cof_segment* segs, uint32_t n_segs, uint64_t n_bases, uint32_t* vs) {
    if (!vs || (!segs && n_segs)) return set_error(COF_E_ARG, "cof_valid_starts: NULL argument");
    const uint64_t words = cof_plane_words(n_bases);
    memset(vs, 0, words * sizeof(uint32_t));
    for (uint32_t k = 0; k < n_segs; k++) {
        const uint64_t a = segs[k].chunk_off, b = a + segs[k].n_owned;
        if (b > n_bases) return set_error(COF_E_ARG, "cof_valid_starts: segment %u ends past the chunk", k);
        if (a == b) continue;
        const uint64_t wa = a >> 5, wb = (b - 1) >> 5;
        if (wa == wb) {
            vs[wa] |= (uint32_t)(((1ull << (b - a)) - 1ull) << (a & 31));
            continue;
        }
        vs[wa] |= ~0u << (a & 31);
#pragma omp parallel for schedule(static) if (wb - wa > (1u << 16))
        for (int64_t w = (int64_t)wa + 1; w < (int64_t)wb; w++) vs[w] = ~0u;
        const uint32_t tail = (uint32_t)(b - (wb << 5));          // 1..32 bits in the last word
        vs[wb] |= tail >= 32 ? ~0u : ((1u << tail) - 1u);
    }
    return COF_OK;
}

cof_status cof_load_chunk(const cof_chunk* host, cof_chunk* dev, cof_stream s) {
    if (!host || !dev || !host->lo || !host->hi || !host->nm || !dev->lo || !dev->hi || !dev->nm)
        return set_error(COF_E_ARG, "cof_load_chunk: NULL argument");
    if (host->n_segs && (!host->vs || !dev->vs))
        return set_error(COF_E_ARG, "cof_load_chunk: multi-segment chunk needs vs planes on both sides");
    size_t bytes = cof_plane_words(host->n_bases) * sizeof(uint32_t);
    cudaStream_t st = (cudaStream_t)s;
    cudaError_t e;
    if ((e = cudaMemcpyAsync(dev->lo, host->lo, bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess ||
        (e = cudaMemcpyAsync(dev->hi, host->hi, bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess ||
        (e = cudaMemcpyAsync(dev->nm, host->nm, bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_error(e, "cof_load_chunk");
    if (host->n_segs && (e = cudaMemcpyAsync(dev->vs, host->vs, bytes, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_error(e, "cof_load_chunk");
    dev->chrom = host->chrom;
    dev->n_segs = host->n_segs;
    dev->start = host->start;
    dev->n_bases = host->n_bases;
    dev->n_owned = host->n_owned;
    dev->segs = host->segs;
    if (!host->n_segs) dev->vs = nullptr;
    return COF_OK;
}

cof_status cof_counts_async(const cof_plan* plan, const void* plan_dev, uint64_t* out_host, cof_stream s) {
    if (!plan || !plan_dev || !out_host) return set_error(COF_E_ARG, "cof_counts_async: NULL argument");
    cudaError_t e = cudaMemcpyAsync(out_host, (const uint8_t*)plan_dev + plan->lay.counters, 3 * sizeof(uint64_t),
                                    cudaMemcpyDeviceToHost, (cudaStream_t)s);
    if (e != cudaSuccess) return cuda_error(e, "cof_counts_async");
    return COF_OK;
}

cof_status cof_read_counts(const cof_plan* plan, const void* plan_dev, uint64_t out[3], cof_stream s) {
    if (!plan || !plan_dev || !out) return set_error(COF_E_ARG, "cof_read_counts: NULL argument");
    uint64_t tmp[3];
    cudaStream_t st = (cudaStream_t)s;
    cudaError_t e = cudaMemcpyAsync(tmp, (const uint8_t*)plan_dev + plan->lay.counters, sizeof tmp,
                                    cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_error(e, "cof_read_counts");
    out[0] = tmp[0]; out[1] = tmp[1]; out[2] = tmp[2];
    return COF_OK;
}

// ------------------------------------------------------------------ FASTA (M2)
struct cof_fasta {
    int fd = -1;
    const char* data = nullptr;
    size_t size = 0;
    struct Rec {
        std::string name;
        size_t seq_off;        // first sequence byte
        size_t seq_end;        // one past the last sequence byte (before next '>')
        uint64_t length;       // bases
        uint64_t line_bases;   // bases per full line (0: single line)
        uint64_t line_bytes;   // bytes per full line incl. newline(s)
        bool regular;          // all lines except the last have line_bases bases
    };
    std::vector<Rec> recs;
};

}  // extern "C"

// One record by a byte-wise line walk from its '>' at d[i] (the general reader: any line
// lengths, blank lines, CR/LF).  Returns the offset of the next record's '>' (or n).
static size_t scan_record(const char* d, size_t n, size_t i, cof_fasta::Rec& r) {
    size_t e = i;
    while (e < n && d[e] != '\n') e++;
    size_t name_end = i + 1;
    while (name_end < e && d[name_end] != ' ' && d[name_end] != '\t' && d[name_end] != '\r') name_end++;
    r.name.assign(d + i + 1, name_end - i - 1);
    r.seq_off = e < n ? e + 1 : n;
    size_t j = r.seq_off;
    r.length = 0; r.line_bases = 0; r.line_bytes = 0; r.regular = true;
    bool seen_short = false;
    while (j < n && d[j] != '>') {
        size_t le = j;
        while (le < n && d[le] != '\n') le++;
        size_t content_end = le;
        if (content_end > j && d[content_end - 1] == '\r') content_end--;
        uint64_t nb = content_end - j;
        size_t lb = (le < n ? le + 1 : le) - j;
        if (r.line_bases == 0 && nb > 0) { r.line_bases = nb; r.line_bytes = lb; }
        else if (nb > 0) {
            if (seen_short || nb > r.line_bases || (nb == r.line_bases && lb != r.line_bytes)) r.regular = false;
            if (nb < r.line_bases) seen_short = true;
        }
        r.length += nb;
        j = le < n ? le + 1 : le;
    }
    r.seq_end = j;
    return j;
}

// The same record by its line geometry alone, for the common layout (every line but the
// last has the first line's length and ending, the last line is not longer, no blank
// lines): the newline count of [seq_off, seq_end) and the byte before every line end are
// checked in parallel instead of walking the bytes.  False: use scan_record.
static bool fast_record(const char* d, size_t n, size_t i, size_t next, cof_fasta::Rec& r) {
    const char* e = (const char*)memchr(d + i, '\n', next - i);
    if (!e) return false;
    size_t name_end = i + 1;
    const size_t hdr_end = (size_t)(e - d);
    while (name_end < hdr_end && d[name_end] != ' ' && d[name_end] != '\t' && d[name_end] != '\r') name_end++;
    r.name.assign(d + i + 1, name_end - i - 1);
    r.seq_off = hdr_end + 1;
    r.seq_end = next;
    r.regular = true;
    const size_t R = r.seq_end - r.seq_off;
    if (R == 0) { r.length = 0; r.line_bases = 0; r.line_bytes = 0; return true; }
    const char* f = (const char*)memchr(d + r.seq_off, '\n', R);
    if (!f) return false;                                   // single line without newline: rare
    const size_t lb = (size_t)(f - d) - r.seq_off + 1;     // first line incl. its '\n'
    const bool crlf = lb >= 2 && d[r.seq_off + lb - 2] == '\r';
    const size_t nb = lb - 1 - (crlf ? 1 : 0);
    if (nb == 0) return false;                              // blank first line
    const size_t F = R / lb, rem = R % lb;
    // the last (partial) line: content, then CR LF / LF, or nothing at the end of the file
    size_t last = rem;
    if (rem) {
        if (d[r.seq_end - 1] == '\n') { last--; if (last && crlf && d[r.seq_end - 2] == '\r') last--; }
        else if (r.seq_end != n) return false;
        if (last == 0) return false;                        // blank line before the next header
    }
    const int64_t FF = (int64_t)F;
    int64_t bad = 0, nl = 0, cr = 0;
    const char* base = d + r.seq_off;
#pragma omp parallel for schedule(static) reduction(+ : bad) if (F > (1u << 16))
    for (int64_t k = 1; k <= FF; k++) {
        const char* le = base + k * lb - 1;
        bad += (*le != '\n') | (crlf && le[-1] != '\r');
    }
    if (bad) return false;
    const int64_t RR = (int64_t)R;
    // newline count (every line break where the geometry puts it) and carriage returns: in an
    // LF record a CR anywhere (e.g. one CRLF line) would be packed as a base -> slow path
#pragma omp parallel for schedule(static) reduction(+ : nl, cr) if (R > (1u << 22))
    for (int64_t k0 = 0; k0 < RR; k0 += 1 << 16) {
        const int64_t k1 = std::min(RR, k0 + (1 << 16));
        int64_t c = 0, c2 = 0;
        for (int64_t k = k0; k < k1; k++) { c += base[k] == '\n'; c2 += base[k] == '\r'; }
        nl += c;
        cr += c2;
    }
    if ((uint64_t)nl != F + (rem && d[r.seq_end - 1] == '\n' ? 1 : 0)) return false;
    if (cr != (crlf ? nl : 0)) return false;
    r.line_bases = nb;
    r.line_bytes = lb;
    r.length = (uint64_t)F * nb + last;
    return true;
}

extern "C" {

cof_status cof_fasta_open(const char* path, cof_fasta** out) {
    if (!path || !out) return set_error(COF_E_ARG, "cof_fasta_open: NULL argument");
    *out = nullptr;
    int fd = open(path, O_RDONLY);
    if (fd < 0) return set_error(COF_E_IO, "cannot open %s", path);
    struct stat st;
    if (fstat(fd, &st) != 0) { close(fd); return set_error(COF_E_IO, "cannot stat %s", path); }
    cof_fasta* fa = new cof_fasta();
    fa->fd = fd;
    fa->size = (size_t)st.st_size;
    if (fa->size) {
        void* m = mmap(nullptr, fa->size, PROT_READ, MAP_PRIVATE, fd, 0);
        if (m == MAP_FAILED) { close(fd); delete fa; return set_error(COF_E_IO, "cannot mmap %s", path); }
        fa->data = (const char*)m;
        madvise(m, fa->size, MADV_WILLNEED);
    }
    const char* d = fa->data;
    const size_t n = fa->size;
    size_t i = 0;
    while (i < n && (d[i] == '\n' || d[i] == '\r')) i++;
    if (i < n && d[i] != '>') {
        cof_fasta_close(fa);
        return set_error(COF_E_IO, "%s: expected '>' at byte %zu", path, i);
    }
    // record starts: '>' at the start of a line, found in parallel blocks with memchr
    const int nt = std::max(1, omp_get_max_threads());
    std::vector<std::vector<size_t>> found(nt);
    const size_t blk = (n - i + nt - 1) / nt;
#pragma omp parallel num_threads(nt)
    {
        const int t = omp_get_thread_num();
        size_t a = i + (size_t)t * blk, b = std::min(n, a + blk);
        while (a < b) {
            const char* g = (const char*)memchr(d + a, '>', b - a);
            if (!g) break;
            const size_t p = (size_t)(g - d);
            if (p == i || d[p - 1] == '\n') found[t].push_back(p);
            a = p + 1;
        }
    }
    std::vector<size_t> starts;
    for (auto& v : found) starts.insert(starts.end(), v.begin(), v.end());
    fa->recs.resize(starts.size());
    for (size_t k = 0; k < starts.size(); k++) {
        const size_t next = k + 1 < starts.size() ? starts[k + 1] : n;
        if (!fast_record(d, n, starts[k], next, fa->recs[k])) scan_record(d, n, starts[k], fa->recs[k]);
    }
    *out = fa;
    return COF_OK;
}

void cof_fasta_close(cof_fasta* fa) {
    if (!fa) return;
    if (fa->data) munmap((void*)fa->data, fa->size);
    if (fa->fd >= 0) close(fa->fd);
    delete fa;
}

uint32_t cof_fasta_count(const cof_fasta* fa) { return fa ? (uint32_t)fa->recs.size() : 0; }
const char* cof_fasta_name(const cof_fasta* fa, uint32_t i) {
    return (fa && i < fa->recs.size()) ? fa->recs[i].name.c_str() : nullptr;
}
uint64_t cof_fasta_length(const cof_fasta* fa, uint32_t i) {
    return (fa && i < fa->recs.size()) ? fa->recs[i].length : 0;
}

cof_status cof_fasta_pack(const cof_fasta* fa, uint32_t i, uint64_t first, uint64_t n, uint32_t* lo,
                          uint32_t* hi, uint32_t* nm) {
    if (!fa || !lo || !hi || !nm) return set_error(COF_E_ARG, "cof_fasta_pack: NULL argument");
    if (i >= fa->recs.size()) return set_error(COF_E_ARG, "cof_fasta_pack: record %u out of range", i);
    const auto& r = fa->recs[i];
    if (first + n > r.length) return set_error(COF_E_ARG, "cof_fasta_pack: range past record end");
    if (r.regular && r.line_bases) {
        // straight from the mapped file: each thread walks its word range line by line
        // (base k is at seq_off + (k / line_bases) * line_bytes + k % line_bases), gathers
        // 32 bases per word and packs them (pack32_ascii); the tail word is N-padded
        const uint64_t LB = r.line_bases, LBY = r.line_bytes;
        const char* seq = fa->data + r.seq_off;
        const int64_t nw = (int64_t)((n + 31) / 32);
#pragma omp parallel if (n > (1u << 20))
        {
            const int nt = omp_get_num_threads(), t = omp_get_thread_num();
            const int64_t per = (nw + nt - 1) / nt;
            const int64_t w0 = std::min(nw, (int64_t)t * per), w1 = std::min(nw, w0 + per);
            if (w0 < w1) {
                uint64_t b = first + (uint64_t)w0 * 32;
                uint64_t line = b / LB, off = b % LB;
                char tmp[32];
                for (int64_t w = w0; w < w1; w++) {
                    const uint64_t want = std::min<uint64_t>(32, n - (uint64_t)w * 32);
                    uint64_t got = 0;
                    if (off + want <= LB) {
                        memcpy(tmp, seq + line * LBY + off, want);
                        got = want;
                        off += want;
                    } else {
                        while (got < want) {
                            const uint64_t take = std::min(want - got, LB - off);
                            memcpy(tmp + got, seq + line * LBY + off, take);
                            got += take;
                            off += take;
                            if (off == LB) { off = 0; line++; }
                        }
                    }
                    if (off == LB) { off = 0; line++; }
                    if (want < 32) memset(tmp + want, 'N', 32 - want);
                    pack32_ascii(tmp, lo[w], hi[w], nm[w]);
                }
            }
        }
        const uint64_t words = cof_plane_words(n);
        for (uint64_t w = (uint64_t)nw; w < words; w++) { lo[w] = 0; hi[w] = 0; nm[w] = ~0u; }
        return COF_OK;
    }
    std::vector<char> buf(n);
    uint64_t b = 0, o = 0;
    for (size_t j = r.seq_off; j < r.seq_end && o < n; j++) {
        char c = fa->data[j];
        if (c == '\n' || c == '\r') continue;
        if (b >= first) buf[o++] = c;
        b++;
    }
    return cof_pack(buf.data(), n, lo, hi, nm);
}

}  // extern "C"

// ------------------------------------------------------------------ collect (M10) / merge
// Decodes one hit key (see cof.h) into a record, building the site string from the host
// planes: '+' reads the window, '-' reads its reverse complement (G6); a compared letter
// is lower-cased where the genome base is not in the guide letter's IUPAC set (G19).
// HIT = cof_hit (L <= 32) or cof_hit64 (L <= 64); windows are 64-bit slices either way.
template <typename HIT>
static cof_status decorate(const cof_plan* plan, const cof_chunk* host, uint64_t key, HIT* h) {
    // char of a (code | N << 2 | mismatch << 3) index: ACGT/N, lower-cased when mismatched
    static const char CH[16] = {'A', 'C', 'G', 'T', 'N', 'N', 'N', 'N', 'a', 'c', 'g', 't', 'n', 'n', 'n', 'n'};
    const uint32_t L = plan->L;
    const uint64_t pos = key >> 32;
    const uint32_t strand = (uint32_t)(key >> 31) & 1u;
    const uint32_t guide = (uint32_t)(key >> 7) & 0xFFFFFFu;
    const uint32_t mm = (uint32_t)key & 127u;
    if (guide >= plan->n_guides || pos + L > host->n_bases || L >= sizeof h->site) return COF_E_STATE;
    // the L-base window as 64-bit slices of the three planes (bit j = base pos + j); the
    // third word is read only when the window reaches into it
    const uint64_t w = pos >> 5;
    const uint32_t sh = (uint32_t)(pos & 31);
    auto win = [&](const uint32_t* pl) -> uint64_t {
        const uint64_t v = ((uint64_t)pl[w + 1] << 32) | pl[w];
        if (sh == 0 || sh + L <= 64) return v >> sh;
        return (v >> sh) | ((uint64_t)pl[w + 2] << (64 - sh));
    };
    const uint64_t lo = win(host->lo), hi = win(host->hi), nm = win(host->nm);
    // mismatched window offsets against the guide in this strand's orientation (bit-parallel)
    const uint64_t* oh = &plan->onehot[((size_t)strand * plan->n_guides + guide) * 5];
    const uint64_t match = (~lo & ~hi & ~nm & oh[0]) | (lo & ~hi & ~nm & oh[1]) | (~lo & hi & ~nm & oh[2]) |
                           (lo & hi & ~nm & oh[3]);
    const uint64_t mis = oh[4] & ~match;
    if ((uint32_t)__builtin_popcountll(mis) != mm) return COF_E_STATE;
    // site read along the strand (G6): '+' = window offset j, '-' = complement of offset L-1-j
    if (strand == 0) {
        for (uint32_t j = 0; j < L; j++)
            h->site[j] = CH[((lo >> j) & 1u) | (((hi >> j) & 1u) << 1) | (((nm >> j) & 1u) << 2) | (((mis >> j) & 1u) << 3)];
    } else {
        for (uint32_t j = 0; j < L; j++) {
            const uint32_t k = L - 1 - j;
            // complement of code c is 3 - c (= c ^ 3); N stays N
            h->site[j] = CH[((((lo >> k) & 1u) | (((hi >> k) & 1u) << 1)) ^ 3u) | (((nm >> k) & 1u) << 2) |
                            (((mis >> k) & 1u) << 3)];
        }
    }
    memset(h->site + L, 0, sizeof h->site - L);
    h->guide = guide;
    if (host->n_segs == 0) {
        h->chrom = host->chrom;
        h->pos = host->start + pos;
    } else {   // chunk coordinate -> (chromosome, chromosome position) through the segment table
        uint32_t lo_k = 0, hi_k = host->n_segs;
        while (hi_k - lo_k > 1) {
            const uint32_t mid = (lo_k + hi_k) / 2;
            if (host->segs[mid].chunk_off <= pos) lo_k = mid;
            else hi_k = mid;
        }
        const cof_segment& sg = host->segs[lo_k];
        if (pos < sg.chunk_off || pos >= sg.chunk_off + sg.n_owned) return COF_E_STATE;
        h->chrom = sg.chrom;
        h->pos = sg.chrom_off + (pos - sg.chunk_off);
    }
    h->strand = strand ? '-' : '+';
    h->mm = (uint8_t)mm;
    return COF_OK;
}

static inline uint64_t sort_key(uint64_t k) { return k >> 7; }   // (pos, strand, guide)

template <typename HIT>
static cof_status collect_t(const char* fn, const cof_plan* plan, const cof_chunk* host, const uint64_t* hits_dev,
                            const uint64_t* host_keys, uint64_t n_hits, HIT* out, cof_stream s) {
    if (!plan || !host || (!out && n_hits) || (!hits_dev && !host_keys && n_hits))
        return set_error(COF_E_ARG, "%s: NULL argument", fn);
    if (!host->lo || !host->hi || !host->nm) return set_error(COF_E_ARG, "%s: host planes are NULL", fn);
    if (plan->L > sizeof out->site - 2)   // cof_hit: L <= 32, cof_hit64: L <= 64
        return set_error(COF_E_ARG, "%s: L = %u does not fit the record (use cof_collect64)", fn, plan->L);
    if (n_hits == 0) return COF_OK;
    std::vector<uint64_t> keys(n_hits);
    if (hits_dev) {
        cudaStream_t st = (cudaStream_t)s;
        cudaError_t e = cudaMemcpyAsync(keys.data(), hits_dev, n_hits * 8, cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) return cuda_error(e, fn);
    } else {
        memcpy(keys.data(), host_keys, n_hits * 8);
    }
    bool sorted = true;
    for (uint64_t i = 1; i < n_hits && sorted; i++) sorted = sort_key(keys[i - 1]) < sort_key(keys[i]);
    if (!sorted) std::sort(keys.begin(), keys.end(), [](uint64_t a, uint64_t b) { return sort_key(a) < sort_key(b); });
    int bad = 0;
#pragma omp parallel for schedule(static) reduction(| : bad) if (n_hits > 4096)
    for (int64_t i = 0; i < (int64_t)n_hits; i++)
        if (decorate(plan, host, keys[i], &out[i]) != COF_OK) bad = 1;
    if (bad) return set_error(COF_E_STATE, "%s: a hit key does not match the plan/chunk (mismatch recount differs)", fn);
    return COF_OK;
}

template <typename HIT>
static inline bool hit_less(const HIT& a, const HIT& b) {
    if (a.chrom != b.chrom) return a.chrom < b.chrom;
    if (a.pos != b.pos) return a.pos < b.pos;
    if (a.strand != b.strand) return a.strand == '+';
    return a.guide < b.guide;
}

template <typename HIT>
static cof_status merge_t(const HIT* const* lists, const uint64_t* lens, uint32_t n_lists, HIT* out) {
    if ((!lists || !lens) && n_lists) return set_error(COF_E_ARG, "cof_merge: NULL argument");
    uint64_t total = 0;
    for (uint32_t i = 0; i < n_lists; i++) {
        if (lens[i] && !lists[i]) return set_error(COF_E_ARG, "cof_merge: list %u is NULL", i);
        for (uint64_t k = 1; k < lens[i]; k++)
            if (hit_less(lists[i][k], lists[i][k - 1])) return set_error(COF_E_ARG, "cof_merge: list %u is not sorted", i);
        total += lens[i];
    }
    if (total && !out) return set_error(COF_E_ARG, "cof_merge: out is NULL");
    // fast path: non-empty lists already in global order (disjoint chunks in genome order)
    {
        bool ordered = true;
        const HIT* prev = nullptr;
        for (uint32_t i = 0; i < n_lists && ordered; i++) {
            if (!lens[i]) continue;
            if (prev && !hit_less(*prev, lists[i][0])) ordered = false;
            prev = &lists[i][lens[i] - 1];
        }
        if (ordered) {
            std::vector<uint64_t> at(n_lists + 1, 0);
            for (uint32_t i = 0; i < n_lists; i++) at[i + 1] = at[i] + lens[i];
            const int64_t CH = 1 << 16;   // records per copy task
            std::vector<std::pair<uint32_t, uint64_t>> tasks;
            for (uint32_t i = 0; i < n_lists; i++)
                for (uint64_t k = 0; k < lens[i]; k += CH) tasks.push_back({i, k});
#pragma omp parallel for schedule(dynamic, 4)
            for (int64_t t = 0; t < (int64_t)tasks.size(); t++) {
                const uint32_t i = tasks[t].first;
                const uint64_t k = tasks[t].second;
                const uint64_t n = std::min<uint64_t>(CH, lens[i] - k);
                memcpy(out + at[i] + k, lists[i] + k, n * sizeof(HIT));
            }
            return COF_OK;
        }
    }
    // k-way merge with a min-heap of list heads (stable across lists for equal keys)
    typedef std::pair<uint32_t, uint64_t> Head;   // (list, index)
    auto cmp = [&](const Head& x, const Head& y) {
        const HIT& a = lists[x.first][x.second];
        const HIT& b = lists[y.first][y.second];
        if (hit_less(a, b)) return false;
        if (hit_less(b, a)) return true;
        return x.first > y.first;
    };
    std::priority_queue<Head, std::vector<Head>, decltype(cmp)> heap(cmp);
    for (uint32_t i = 0; i < n_lists; i++) if (lens[i]) heap.push({i, 0});
    uint64_t o = 0;
    while (!heap.empty()) {
        Head h = heap.top();
        heap.pop();
        out[o++] = lists[h.first][h.second];
        if (h.second + 1 < lens[h.first]) heap.push({h.first, h.second + 1});
    }
    return COF_OK;
}


extern "C" {

cof_status cof_collect(const cof_plan* plan, const cof_chunk* host, const uint64_t* hits_dev,
                       const uint64_t* host_keys, uint64_t n_hits, cof_hit* out, cof_stream s) {
    return collect_t("cof_collect", plan, host, hits_dev, host_keys, n_hits, out, s);
}

cof_status cof_collect64(const cof_plan* plan, const cof_chunk* host, const uint64_t* hits_dev,
                         const uint64_t* host_keys, uint64_t n_hits, cof_hit64* out, cof_stream s) {
    return collect_t("cof_collect64", plan, host, hits_dev, host_keys, n_hits, out, s);
}

cof_status cof_merge(const cof_hit* const* lists, const uint64_t* lens, uint32_t n_lists, cof_hit* out) {
    return merge_t(lists, lens, n_lists, out);
}

cof_status cof_merge64(const cof_hit64* const* lists, const uint64_t* lens, uint32_t n_lists, cof_hit64* out) {
    return merge_t(lists, lens, n_lists, out);
}

}  // extern "C"
