/*
 * cof.h -- C ABI of the B200-native Cas-OFFinder hot path (libcof.so).
 *
 * Paper: Jin & Vetter, "Experience Migrating OpenCL to SYCL: A Case Study on Searches
 * for Potential Off-Target Sites of Cas9 RNA-Guided Endonucleases on AMD GPUs";
 * "P:Lnn" = line nn of /root/reference/PAPER.md.  The calls follow the paper's
 * problem statement: the host divides the genome into chunks that fit device
 * memory, a "search" kernel selects the sites carrying a PAM, a "compare" kernel counts
 * mismatched bases for every query, and the host collects "chromosome number, position,
 * direction, the number of mismatched bases and potential off-target DNA sequence with
 * mismatched bases".  Readings of points the paper leaves open are listed in DESIGN.md
 * §2 (G1..G19) and referenced below.
 *
 * Conventions (all calls):
 *  - Return COF_OK (0) or a negative cof_status; never throw, never abort.  On error
 *    cof_last_error() returns a thread-local message.
 *  - Every buffer is caller-owned; the library never frees caller memory.  "dev" means
 *    a device pointer of the calling thread's current CUDA device, "host" a host pointer
 *    (pinned for the async copies to be truly asynchronous).
 *  - cof_stream is a cudaStream_t passed as an opaque pointer (NULL = legacy stream).
 *    Calls are asynchronous on that stream unless they return a host-side count, in
 *    which case they synchronize it.
 *  - No torch types cross this boundary; the Python binding passes data_ptr()s.
 */
#ifndef COF_H
#define COF_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t cof_status;
#define COF_OK          0
#define COF_E_ARG      (-1)   /* bad argument: non-IUPAC letter, length mismatch, L>64, NULL, ... */
#define COF_E_CAPACITY (-2)   /* output buffer too small; the needed count is returned */
#define COF_E_CUDA     (-3)   /* CUDA runtime error (message has the CUDA error string) */
#define COF_E_STATE    (-4)   /* plan / chunk / workspace mismatch */
#define COF_E_IO       (-5)   /* file could not be read / parsed */

/* Longest pattern / guide (two 32-bit plane words per window).  The
 * paper fixes no bound (Listing 1 loops over plen).  Patterns with L <= 32 use
 * one-word windows and the 56-byte cof_hit; 32 < L <= 64 use two-word windows and the
 * 88-byte cof_hit64 (cof_collect64 / cof_decorate64 / cof_merge64). */
#define COF_MAX_L 64

/* Pass as a count to cof_compare / cof_sort_hits to use the count the previous call
 * left in the plan's device workspace (no host round trip between kernels). */
#define COF_COUNT_ON_DEVICE UINT64_MAX

typedef void *cof_stream;

const char *cof_last_error(void);
const char *cof_version(void);
/* Number of CUDA kernels this library has launched in this process (monotone). */
uint64_t cof_launch_count(void);
/* Host threads of the library's OpenMP regions (packing, collection, merge); n <= 0 keeps
 * the current setting.  (torchrun sets OMP_NUM_THREADS=1 for every rank; a multi-GPU
 * caller shares the node's cores among its ranks instead.)  Returns the setting in force. */
int cof_set_host_threads(int n);

/* ------------------------------------------------------------------ plan (M1)
 * The input specification: a search pattern of length L (guide Ns + PAM, e.g.
 * "NNNNNNNNNNNNNNNNNNNNNRG") and n queries ("guides") of the same length, each with its
 * own maximum mismatch count (P:L158 via [17]; Listing 1 parameters P:L185-L188).
 *  pattern   NUL-terminated IUPAC string (ACGTRYSWKMBDHVN, case-insensitive), 1<=L<=64.
 *  guides    n_guides NUL-terminated IUPAC strings of length L; 'N' positions are not
 *            compared (the -1-terminated index list; reading G7).
 *  max_mm    n_guides thresholds, each <= L; a site is a hit iff #mismatches <= max_mm
 *            (P:L225).
 *  out       receives a host-only, immutable plan (thread-safe to share read-only).
 * Errors: COF_E_ARG for a non-IUPAC letter (G18), guide length != L (G11), L>64, max_mm > L, a
 * guide with 64 compared (non-N) letters, n_guides == 0 or > 2^24, NULL pointers.  For
 * L > 32 the comparer is always the pair-table one (cof_set_comparer's popc variant
 * needs L <= 32).  The plan reverse-complements pattern and
 * guides for the '-' strand and groups guides by compared-position mask. */
typedef struct cof_plan cof_plan;
cof_status cof_plan_create(const char *pattern, uint32_t n_guides, const char *const *guides,
                           const uint8_t *max_mm, cof_plan **out);
void       cof_plan_destroy(cof_plan *plan);
uint32_t   cof_plan_length(const cof_plan *plan);        /* L */
uint32_t   cof_plan_n_guides(const cof_plan *plan);
/* Bytes of the device-side plan (guide tables + counters).  One plan_dev per
 * (device, stream) in flight: it holds the counters find/compare/sort exchange. */
size_t     cof_plan_device_bytes(const cof_plan *plan);
/* Async H2D of the guide tables into plan_dev (>= cof_plan_device_bytes, 256-B aligned). */
cof_status cof_plan_upload(const cof_plan *plan, void *plan_dev, cof_stream s);

/* ------------------------------------------------------------------ chunk (M3, M4)
 * A chunk is the unit the device works on ("divides the genome data into chunks that
 * can fit the memory of a heterogeneous device").  It holds n_bases bases stored as three
 * bit-planes of uint32 words (bit p&31 of word p>>5 is base p): lo/hi = 2-bit code A=00
 * C=01 G=10 T=11 (lo = bit 0), nm = 1 for any non-ACGT letter (then lo=hi=0), readings
 * G2/G4; the "2-bit sequence format" of P:L289.  Each plane has cof_plane_words(n_bases)
 * words; words past the last base have nm = all-ones.  Positions inside a chunk are
 * chunk coordinates (< 2^32).
 *
 * Single-segment chunk (n_segs == 0): bases [start, start + n_bases) of chromosome `chrom`;
 * window starts [0, n_owned) belong to it, n_bases = min(n_owned + L - 1, chrom_len - start)
 * (chunks of one chromosome overlap by L-1, reading G12).
 * Multi-segment chunk (n_segs > 0): several chromosome pieces laid back to back (e.g. a
 * whole genome or one GPU's shard); segs[k] (HOST array, ascending chunk_off) says which
 * chromosome piece starts at chunk offset chunk_off and which window starts it owns; vs is
 * the valid-start plane (bit p = 1 iff start p is owned, see cof_valid_starts), so no window
 * spanning two pieces is ever reported. */
typedef struct {
    uint32_t chrom;        /* chromosome index */
    uint32_t reserved;
    uint64_t chunk_off;    /* chunk offset of the piece's first base */
    uint64_t chrom_off;    /* chromosome offset of that base */
    uint64_t n_owned;      /* window starts [chunk_off, chunk_off + n_owned) belong to the chunk */
} cof_segment;

typedef struct {
    uint32_t chrom;        /* single-segment: chromosome index (FASTA / caller order) */
    uint32_t n_segs;       /* 0 = single segment; else number of entries in segs */
    uint64_t start;        /* single-segment: 0-based chromosome offset of base 0 */
    uint64_t n_bases;
    uint64_t n_owned;      /* owned window starts (single: [0, n_owned); multi: total) */
    uint32_t *lo, *hi, *nm;
    uint32_t *vs;          /* multi-segment: valid-start plane (same word count); else NULL */
    const cof_segment *segs;   /* multi-segment: HOST segment table (collect, valid starts) */
} cof_chunk;

uint64_t   cof_plane_words(uint64_t n_bases);
/* Host pack (OpenMP): n ASCII bases -> planes of cof_plane_words(n) words each.
 * Upper/lower case are equal; any non-ACGT byte becomes N (G2, G4). */
cof_status cof_pack(const char *ascii, uint64_t n, uint32_t *lo, uint32_t *hi, uint32_t *nm);
/* Host unpack (inverse, canonical form: "ACGTN" upper-case), for checks and output. */
cof_status cof_unpack(const uint32_t *lo, const uint32_t *hi, const uint32_t *nm,
                      uint64_t first, uint64_t n, char *ascii);
/* Valid-start plane of a multi-segment chunk: bit p = 1 iff p lies in
 * [segs[k].chunk_off, segs[k].chunk_off + segs[k].n_owned) for some k (host, OpenMP).
 * vs has cof_plane_words(n_bases) words.  COF_E_ARG if a segment leaves the chunk. */
cof_status cof_valid_starts(const cof_segment *segs, uint32_t n_segs, uint64_t n_bases, uint32_t *vs);
/* Async H2D of the host planes (and vs, if both chunks have one) into the device buffers
 * of dev (cof_plane_words(host->n_bases) words each); copies the metadata fields and the
 * segs pointer too.  (Table III.) */
cof_status cof_load_chunk(const cof_chunk *host, cof_chunk *dev, cof_stream s);
/* N runs of a chunk (host): the maximal [begin, end) intervals of N bases (nm bit set)
 * among bases [0, n_bases), ascending, as pairs runs[2i], runs[2i+1].  *n_runs = the count;
 * COF_E_CAPACITY (contents past cap unspecified) if it exceeds cap pairs. */
cof_status cof_n_runs(const uint32_t *nm, uint64_t n_bases, uint64_t *runs, uint64_t cap,
                      uint64_t *n_runs);
/* cof_load_chunk with the sparse planes built on the device: H2D of lo/hi only (1/4 B per
 * base), dev->nm rebuilt from the n_runs N runs (cof_n_runs of the chunk) and, for a
 * multi-segment chunk, dev->vs from host->segs (the owned-start intervals) by small kernels
 * on stream s.  host->nm / host->vs are not read.  The device planes equal what
 * cof_load_chunk would copy.  COF_E_ARG for runs that are not ascending intervals inside
 * the chunk or a segment that leaves it. */
cof_status cof_load_chunk_runs(const cof_chunk *host, const uint64_t *runs, uint64_t n_runs,
                               cof_chunk *dev, cof_stream s);
/* The same with the two halves on two streams: the lo/hi DMA on s_copy, the nm / vs fill
 * kernels on s_fill (e.g. the stream that runs this chunk's kernels, so the fills are not
 * queued behind a copy engine waiting on a persistent kernel, and the DMA queue holds
 * DMA only).  The caller orders s_fill's later work after s_copy (an event) before
 * reading lo/hi.  Arguments, ownership and errors as cof_load_chunk_runs. */
cof_status cof_load_chunk_runs_split(const cof_chunk *host, const uint64_t *runs, uint64_t n_runs,
                                     cof_chunk *dev, cof_stream s_copy, cof_stream s_fill);

/* ------------------------------------------------------------------ FASTA (M2)
 * Minimal indexed FASTA reader ("single- or multi-sequence data format"):
 * mmap + per-record line layout; packs any base range straight into planes. */
typedef struct cof_fasta cof_fasta;
cof_status cof_fasta_open(const char *path, cof_fasta **out);
void       cof_fasta_close(cof_fasta *fa);
uint32_t   cof_fasta_count(const cof_fasta *fa);
const char *cof_fasta_name(const cof_fasta *fa, uint32_t i);
uint64_t   cof_fasta_length(const cof_fasta *fa, uint32_t i);
/* Pack bases [first, first+n) of record i into planes (cof_plane_words(n) words each). */
cof_status cof_fasta_pack(const cof_fasta *fa, uint32_t i, uint64_t first, uint64_t n,
                          uint32_t *lo, uint32_t *hi, uint32_t *nm);

/* ------------------------------------------------------------------ UCSC .2bit (f2)
 * The packed genome format genomes are distributed in (hg38.2bit): 4 bases per byte, N
 * and soft-mask runs as block lists.  Same interface as the FASTA reader: records are the
 * file's sequences in index order; cof_2bit_pack writes bases [first, first+n) of record
 * i into planes of cof_plane_words(n) words (N blocks -> nm = 1, lo = hi = 0; soft-mask
 * ignored, reading G4).  COF_E_IO for a malformed or truncated file (checked at open),
 * COF_E_ARG for a range past the record end. */
typedef struct cof_twobit cof_twobit;
cof_status cof_2bit_open(const char *path, cof_twobit **out);
void       cof_2bit_close(cof_twobit *t);
uint32_t   cof_2bit_count(const cof_twobit *t);
const char *cof_2bit_name(const cof_twobit *t, uint32_t i);
uint64_t   cof_2bit_length(const cof_twobit *t, uint32_t i);
cof_status cof_2bit_pack(const cof_twobit *t, uint32_t i, uint64_t first, uint64_t n,
                         uint32_t *lo, uint32_t *hi, uint32_t *nm);

/* ------------------------------------------------------------------ finder (M5, M6)
 * The "search" kernel (signature Table VI): for every owned window
 * start p (single segment: p < n_owned; multi: vs bit set) with p+L <= n_bases, '+'
 * passes iff every non-N pattern letter P[j] contains
 * base(p+j); '-' passes iff the reverse-complemented pattern does (G3, G10).  Passing
 * starts are compacted in ascending order into one list per strand (chunk-relative
 * uint32).  The paper compacts with an unordered atomic counter (Table V);
 * here an ordered two-pass compaction (count, one grid-wide exchange, write) keeps the
 * lists sorted.
 *  workspace  dev, >= cof_find_workspace_bytes(dev->n_bases) bytes (per-CTA totals, a
 *             grid barrier counter and the pass-1 PAM masks, 8 bytes per plane word).
 *  items_cap  capacity of each list; n_owned always suffices.
 *  n_fwd/n_rev  host outputs; if both are NULL the call does not synchronize and the
 *             counts stay in plan_dev for cof_compare(COF_COUNT_ON_DEVICE).
 * COF_E_CAPACITY: a list overflowed; n_fwd and n_rev hold the needed counts. */
size_t     cof_find_workspace_bytes(uint64_t n_bases);
cof_status cof_find_pam(const cof_plan *plan, void *plan_dev, const cof_chunk *dev,
                        void *workspace, uint32_t *items_fwd, uint32_t *items_rev,
                        uint64_t items_cap, uint64_t *n_fwd, uint64_t *n_rev, cof_stream s);

/* ------------------------------------------------------------------ comparer (M8, M9)
 * The "compare" kernel (Listing 1): for every item and every guide,
 * mm = #compared positions whose genome base is not in the guide letter's IUPAC set
 * ('-' items use the reverse-complemented guide aligned to the same '+' window,
 * P:L231-L236); emit iff mm <= max_mm.  Emission is a
 * warp-aggregated atomic append of a 64-bit key
 *     key = pos << 32 | strand << 31 | guide << 7 | mm      (strand 0 = '+', 1 = '-')
 * so that integer order is (pos, '+' before '-', guide) (G13).
 *  n_fwd/n_rev  item counts, or COF_COUNT_ON_DEVICE to use the finder's device counts.
 *  hits     dev, capacity hits_cap keys; n_hits host output (NULL: no sync, the count
 *           stays in plan_dev).  Order of hits is unspecified (see cof_sort_hits).
 * COF_E_CAPACITY: *n_hits holds the needed count; re-run with a larger buffer. */
cof_status cof_compare(const cof_plan *plan, void *plan_dev, const cof_chunk *dev,
                       const uint32_t *items_fwd, uint64_t n_fwd,
                       const uint32_t *items_rev, uint64_t n_rev,
                       uint64_t *hits, uint64_t hits_cap, uint64_t *n_hits, cof_stream s);

/* Comparer implementation for cof_compare (process-wide): 0 = "popc" (POPC per
 * comparison), 1 = "table" (bit-sliced pair tables on the ALU, default).  Both return the
 * same hits.  COF_E_ARG for another value.  (Env COF_COMPARER=popc|table sets the initial
 * choice.)  The fused path (cof_find_compare) is the table comparer's. */
cof_status cof_set_comparer(int impl);

/* ------------------------------------------------------------------ fused find + compare
 * the search and compare kernels of P:L29 without the host hand-off and
 * without the item lists: the finder (pass 1 only) writes per-word PAM masks into the
 * workspace and the comparer expands them itself (shared-memory queue) before the table
 * comparison.  Same hits as cof_find_pam + cof_compare (same key format, unordered); the
 * item counts land in plan_dev (cof_read_counts).  Each launch keeps its guide blocks
 * resident in shared memory; larger guide sets run several launches per strand that
 * re-expand the masks (up to 512 launches per strand, cof_find_compare_supported;
 * otherwise COF_E_ARG).  Requires the table comparer (cof_set_comparer(1), the default).
 *  workspace  dev, >= cof_find_compare_workspace_bytes(dev->n_bases) bytes. */
int        cof_find_compare_supported(const cof_plan *plan);
size_t     cof_find_compare_workspace_bytes(uint64_t n_bases);
/* = cof_search_single when cof_single_supported(plan), else cof_find_masks +
 * cof_compare_masks.  Same arguments as cof_compare_masks. */
cof_status cof_find_compare(const cof_plan *plan, void *plan_dev, const cof_chunk *dev, void *workspace,
                            uint64_t *hits, uint64_t hits_cap, uint64_t *n_hits, cof_stream s);
/* Single pass (SURVEY §8(f) f1 as one streaming kernel, single.cu): the planes stream
 * through shared memory once; each tile's PAM test (both strands) feeds per-warp queues
 * of sites with their 32-base windows, which are compared against all guides of the
 * launch: a necessary-condition filter (number of mismatched position pairs <= t, from
 * one 32-bit shared-memory lookup per pair and 32 guides) and the exact count of every
 * survivor, hits appended warp-aggregated.  No item list,
 * no mask array, no window gather.  Same hits as cof_find_pam + cof_compare (same key
 * format, unordered); item counts land in plan_dev.  Needs every compared position of
 * both strands inside one 31-position window (L <= 32 patterns) and the table comparer;
 * COF_E_ARG otherwise.  Guide sets larger than one launch's shared-memory tables (~1,500
 * 20-nt guides) run several launches, each re-streaming the planes.
 * cof_single_supported(plan) = 1 when the shape fits AND the filter is selective (every
 * threshold at least 3 below the number of position pairs); COF_SINGLE=1 / 0 overrides.
 *  workspace  dev, >= cof_find_compare_workspace_bytes(dev->n_bases) bytes (tile tickets). */
int        cof_single_supported(const cof_plan *plan);
cof_status cof_search_single(const cof_plan *plan, void *plan_dev, const cof_chunk *dev, void *workspace,
                             uint64_t *hits, uint64_t hits_cap, uint64_t *n_hits, cof_stream s);
/* The search kernel's pass 1 alone: PAM masks of every plane word, both strands, into the
 * workspace ({fwd, rev} 32-bit masks per plane word, bit b = window start 32w + b);
 * item counts into plan_dev.  Asynchronous. */
cof_status cof_find_masks(const cof_plan *plan, void *plan_dev, const cof_chunk *dev, void *workspace,
                          cof_stream s);
/* The comparer over those masks (n_hits: host count, NULL = no sync). */
cof_status cof_compare_masks(const cof_plan *plan, void *plan_dev, const cof_chunk *dev, void *workspace,
                             uint64_t *hits, uint64_t hits_cap, uint64_t *n_hits, cof_stream s);

/* ------------------------------------------------------------------ sort (M10, K3)
 * Deterministic order of the hit keys (the paper's atomics are unordered):
 * stable LSD radix sort on the device of the key bits that vary for this chunk.
 *  hits/tmp dev buffers of >= n_hits keys; the sorted keys end up in hits.
 *  workspace dev, >= cof_sort_workspace_bytes(cap) bytes.
 *  n_hits   count or COF_COUNT_ON_DEVICE (the comparer's count, clamped to cap). */
size_t     cof_sort_workspace_bytes(uint64_t cap);
cof_status cof_sort_hits(const cof_plan *plan, void *plan_dev, const cof_chunk *dev,
                         uint64_t *hits, uint64_t *tmp, uint64_t cap, uint64_t n_hits,
                         void *workspace, cof_stream s);

/* Device counters of plan_dev: out[0]=n_fwd, out[1]=n_rev, out[2]=n_hits (synchronizes). */
cof_status cof_read_counts(const cof_plan *plan, const void *plan_dev, uint64_t out[3],
                           cof_stream s);
/* The same three counters copied asynchronously on stream s into out_host (caller-owned,
 * ideally pinned; valid once the stream reaches this point -- record an event after it).
 * No synchronisation: lets a pipelined caller read chunk j's counts while chunk j+1 runs. */
cof_status cof_counts_async(const cof_plan *plan, const void *plan_dev, uint64_t *out_host,
                            cof_stream s);

/* ------------------------------------------------------------------ collect (M10)
 * One output record: guide index, chromosome, 0-based '+'-strand chromosome
 * position (G5; chunk coordinates are mapped back through the segment table),
 * direction, #mismatches, and the L-letter site read along its strand (G6) with
 * mismatched compared letters in lower case (G19). */
typedef struct {
    uint32_t guide;
    uint32_t chrom;
    uint64_t pos;
    char     strand;   /* '+' or '-' */
    uint8_t  mm;
    char     site[34]; /* NUL-terminated */
} cof_hit;

/* The same record for patterns with 32 < L <= 64 (site up to 64 letters). */
typedef struct {
    uint32_t guide;
    uint32_t chrom;
    uint64_t pos;
    char     strand;   /* '+' or '-' */
    uint8_t  mm;
    char     site[66]; /* NUL-terminated */
} cof_hit64;

/* D2H the n_hits keys from hits_dev (stream s), order them (host sort if they are not
 * already sorted), and decorate them from the HOST planes of the same chunk.
 * out must hold n_hits records; it is sorted by (pos, strand, guide).
 * If hits_dev is NULL, keys are read from host_keys instead (already on the host). */
cof_status cof_collect(const cof_plan *plan, const cof_chunk *host, const uint64_t *hits_dev,
                       const uint64_t *host_keys, uint64_t n_hits, cof_hit *out, cof_stream s);
/* cof_collect for plans with L > 32 (also accepts L <= 32). */
cof_status cof_collect64(const cof_plan *plan, const cof_chunk *host, const uint64_t *hits_dev,
                         const uint64_t *host_keys, uint64_t n_hits, cof_hit64 *out, cof_stream s);

/* The same decoration on the device: n_hits (sorted) keys of hits_dev -> n_hits records in
 * the DEVICE buffer out_dev (same order; n_hits = COF_COUNT_ON_DEVICE: the count of the
 * last compare in plan_dev, clamped to cap), one thread per hit, from the device planes of
 * the chunk and the guide masks in plan_dev; dev->segs (host) is copied into workspace
 * (>= cof_decorate_workspace_bytes(dev->n_segs) device bytes).  Asynchronous; a key that
 * does not match the chunk/plan sets a flag that cof_decorate_check reports (COF_E_STATE,
 * synchronizes).  The caller copies the records to the host (pinned memory: no staging). */
size_t     cof_decorate_workspace_bytes(uint32_t n_segs);
cof_status cof_decorate(const cof_plan *plan, const void *plan_dev, const cof_chunk *dev,
                        const uint64_t *hits_dev, uint64_t n_hits, uint64_t cap, cof_hit *out_dev,
                        void *workspace, cof_stream s);
/* cof_decorate for plans with L > 32 (also accepts L <= 32): cof_hit64 records. */
cof_status cof_decorate64(const cof_plan *plan, const void *plan_dev, const cof_chunk *dev,
                          const uint64_t *hits_dev, uint64_t n_hits, uint64_t cap, cof_hit64 *out_dev,
                          void *workspace, cof_stream s);
cof_status cof_decorate_check(const void *workspace, cof_stream s);

/* k-way merge of sorted lists into out (sum of lens records), order (chrom, pos,
 * strand, guide) (G13).  Lists from disjoint chunks merge by concatenation. */
cof_status cof_merge(const cof_hit *const *lists, const uint64_t *lens, uint32_t n_lists,
                     cof_hit *out);
cof_status cof_merge64(const cof_hit64 *const *lists, const uint64_t *lens, uint32_t n_lists,
                       cof_hit64 *out);

#ifdef __cplusplus
}
#endif
#endif /* COF_H */
