/*
 * cof_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously correct CPU brute-force scanner for the Cas-OFFinder
 * hot path (PAM "search" + mismatch "compare").  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load it.  It shares no
 * code, table or header with the CUDA path (paper_conf_socc_jinv23_b200/csrc) and
 * works on ASCII characters, not on packed bit-planes.
 *
 * Paper = /root/reference/PAPER.md (Jin & Vetter, "Experience Migrating OpenCL to
 * SYCL ..."); "P:Lnn" = line nn of that file.
 *
 * What it computes:
 *   for every chromosome c, every window start 0 <= p <= len_c - L, strand s in {+,-}:
 *     W = canon(seq_c[p, p+L))                   canon: upper-case, non-ACGT -> 'N'  (readings G2, G4)
 *     S = W if s = '+', else reverse-complement(W)                                   (reading G6)
 *     PAM ("search" kernel):  for all j with P[j] != 'N':  S[j] in IUPAC(P[j])
 *     compare (Listing 1): for each guide i
 *        mm = #{ j : g_i[j] != 'N'  and  S[j] not in IUPAC(g_i[j]) }   (non-N index list, P:L207-L208;
 *                                                                         mismatch rows P:L209-L221)
 *        emit if mm <= t_i  (inclusive, P:L225 / P:L242)
 *        site[j] = S[j], lower-cased where g_i[j] != 'N' and it mismatched (output fields)
 *   order: (chromosome, position, '+' before '-', guide)            (reading G13)
 * A genome 'N' is in no IUPAC set, so it fails every non-N pattern letter and is a
 * mismatch against every non-N guide letter (reading G2).  The early exit once
 * mm > t cannot change which hits are emitted and is kept.
 *
 * Parallelism: OpenMP over fixed position blocks; each block's hits are produced in
 * (pos, strand, guide) order and blocks are concatenated in order, so the output is
 * already sorted and identical for any thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Longest pattern the oracle accepts (reading G11: guide length = pattern length).  The
 * paper fixes no bound; 64 covers the CUDA path's two-word windows. */
#define COF_ORACLE_MAX_L 64

typedef struct {
    int32_t guide;
    int32_t chrom;
    int64_t pos;      /* 0-based leftmost base of the window on the '+' strand (reading G5) */
    char strand;      /* '+' or '-' */
    int8_t mm;
    char site[66];    /* NUL-terminated, length L (L <= COF_ORACLE_MAX_L) */
} oracle_hit;

/* ---- IUPAC nucleotide codes, written out as the nomenclature defines them ---- */
/* Returns 1 if genome base b (one of 'A','C','G','T','N') is a member of the set
 * denoted by IUPAC code x (upper case).  'N' as a genome base is in no set. */
static int iupac_contains(char x, char b)
{
    if (b != 'A' && b != 'C' && b != 'G' && b != 'T')
        return 0;
    switch (x) {
    case 'A': return b == 'A';
    case 'C': return b == 'C';
    case 'G': return b == 'G';
    case 'T': return b == 'T';
    case 'R': return b == 'A' || b == 'G';               /* puRine            */
    case 'Y': return b == 'C' || b == 'T';               /* pYrimidine        */
    case 'S': return b == 'C' || b == 'G';               /* Strong            */
    case 'W': return b == 'A' || b == 'T';               /* Weak              */
    case 'K': return b == 'G' || b == 'T';               /* Keto              */
    case 'M': return b == 'A' || b == 'C';               /* aMino             */
    case 'B': return b != 'A';                           /* not A             */
    case 'D': return b != 'C';                           /* not C             */
    case 'H': return b != 'G';                           /* not G             */
    case 'V': return b != 'T';                           /* not T             */
    case 'N': return 1;                                  /* aNy               */
    default:  return 0;
    }
}

static int is_iupac_code(char x)
{
    return x && strchr("ACGTRYSWKMBDHVN", x) != NULL;
}

static char upper(char c)
{
    return (c >= 'a' && c <= 'z') ? (char)(c - 'a' + 'A') : c;
}

/* canon(): upper-case; anything that is not A/C/G/T becomes 'N' (readings G2, G4, G19). */
static char canon(char c)
{
    c = upper(c);
    return (c == 'A' || c == 'C' || c == 'G' || c == 'T') ? c : 'N';
}

static char complement_base(char b)
{
    switch (b) {
    case 'A': return 'T';
    case 'C': return 'G';
    case 'G': return 'C';
    case 'T': return 'A';
    default:  return 'N';
    }
}

static char lower(char c)
{
    return (c >= 'A' && c <= 'Z') ? (char)(c - 'A' + 'a') : c;
}

/* exported for the truth-table pins */
int cof_oracle_contains(char code, char base) { return iupac_contains(upper(code), canon(base)); }
char cof_oracle_canon(char c) { return canon(c); }
char cof_oracle_complement_base(char b) { return complement_base(canon(b)); }

typedef struct {
    oracle_hit *v;
    int64_t n, cap;
} hitvec;

static int push(hitvec *h, const oracle_hit *x)
{
    if (h->n == h->cap) {
        int64_t nc = h->cap ? h->cap * 2 : 64;
        oracle_hit *nv = (oracle_hit *)realloc(h->v, (size_t)nc * sizeof(oracle_hit));
        if (!nv) return -1;
        h->v = nv;
        h->cap = nc;
    }
    h->v[h->n++] = *x;
    return 0;
}

/* Builds the strand-s reading S of the window at p: S = W ('+') or revcomp(W) ('-'). */
static void window_reading(const char *seq, int64_t p, int L, char strand, char *S)
{
    char W[COF_ORACLE_MAX_L + 1];
    for (int j = 0; j < L; j++)
        W[j] = canon(seq[p + j]);
    if (strand == '+') {
        for (int j = 0; j < L; j++) S[j] = W[j];
    } else {
        for (int j = 0; j < L; j++) S[j] = complement_base(W[L - 1 - j]);
    }
    S[L] = 0;
}

static int pam_ok(const char *S, const char *P, int L)
{
    for (int j = 0; j < L; j++)
        if (P[j] != 'N' && !iupac_contains(P[j], S[j]))
            return 0;
    return 1;
}

static int validate(const char *pattern, int n_guides, const char *const *guides,
                    const int32_t *max_mm, int *Lout)
{
    int L = (int)strlen(pattern);
    if (L < 1 || L > COF_ORACLE_MAX_L) return -1;
    for (int j = 0; j < L; j++)
        if (!is_iupac_code(upper(pattern[j]))) return -1;
    for (int i = 0; i < n_guides; i++) {
        if ((int)strlen(guides[i]) != L) return -1;
        for (int j = 0; j < L; j++)
            if (!is_iupac_code(upper(guides[i][j]))) return -1;
        if (max_mm[i] < 0) return -1;
    }
    *Lout = L;
    return 0;
}

/*
 * Full search.  seqs[c] has lens[c] ASCII bytes.  Window starts p in [begin[c], end[c])
 * are scanned (begin/end may be NULL = whole chromosome; they are clipped to the
 * valid range 0 <= p <= len-L).  On success returns the number of hits and sets
 * *out (free with cof_oracle_free); returns -1 on bad arguments, -2 on OOM.
 */
int64_t cof_oracle_search(int32_t n_chrom, const char *const *seqs, const int64_t *lens,
                          const int64_t *begin, const int64_t *end,
                          const char *pattern_in, int32_t n_guides,
                          const char *const *guides_in, const int32_t *max_mm,
                          int32_t n_threads, oracle_hit **out)
{
    int L;
    *out = NULL;
    if (validate(pattern_in, n_guides, guides_in, max_mm, &L)) return -1;
    char P[COF_ORACLE_MAX_L + 1];
    for (int j = 0; j < L; j++) P[j] = upper(pattern_in[j]);
    P[L] = 0;
    char (*G)[COF_ORACLE_MAX_L + 1] = (char (*)[COF_ORACLE_MAX_L + 1])malloc((size_t)(n_guides ? n_guides : 1) * (COF_ORACLE_MAX_L + 1));
    if (!G) return -2;
    for (int i = 0; i < n_guides; i++) {
        for (int j = 0; j < L; j++) G[i][j] = upper(guides_in[i][j]);
        G[i][L] = 0;
    }

    const int64_t BLOCK = 1 << 12;
    hitvec all = {0, 0, 0};
    int err = 0;
    for (int32_t c = 0; c < n_chrom && !err; c++) {
        int64_t lo = 0, hi = lens[c] - L + 1;       /* valid starts: 0 <= p <= len-L */
        if (begin && begin[c] > lo) lo = begin[c];
        if (end && end[c] < hi) hi = end[c];
        if (hi <= lo) continue;
        int64_t nblocks = (hi - lo + BLOCK - 1) / BLOCK;
        hitvec *bv = (hitvec *)calloc((size_t)nblocks, sizeof(hitvec));
        if (!bv) { err = 1; break; }
#ifdef _OPENMP
        if (n_threads > 0) omp_set_num_threads(n_threads);
#pragma omp parallel for schedule(dynamic, 1)
#endif
        for (int64_t b = 0; b < nblocks; b++) {
            int64_t p0 = lo + b * BLOCK, p1 = p0 + BLOCK < hi ? p0 + BLOCK : hi;
            char S[COF_ORACLE_MAX_L + 1];
            for (int64_t p = p0; p < p1; p++) {
                for (int s = 0; s < 2; s++) {
                    char strand = s == 0 ? '+' : '-';
                    window_reading(seqs[c], p, L, strand, S);
                    if (!pam_ok(S, P, L)) continue;
                    for (int i = 0; i < n_guides; i++) {
                        int mm = 0;
                        for (int j = 0; j < L; j++) {
                            if (G[i][j] == 'N') continue;          /* not in comp_index */
                            if (!iupac_contains(G[i][j], S[j])) {
                                mm++;
                                if (mm > max_mm[i]) break;
                            }
                        }
                        if (mm > max_mm[i]) continue;
                        oracle_hit h;
                        memset(&h, 0, sizeof h);
                        h.guide = i; h.chrom = c; h.pos = p; h.strand = strand; h.mm = (int8_t)mm;
                        for (int j = 0; j < L; j++) {
                            int mis = G[i][j] != 'N' && !iupac_contains(G[i][j], S[j]);
                            h.site[j] = mis ? lower(S[j]) : S[j];
                        }
                        h.site[L] = 0;
                        if (push(&bv[b], &h)) err = 1;
                    }
                }
            }
        }
        for (int64_t b = 0; b < nblocks; b++) {
            for (int64_t k = 0; k < bv[b].n && !err; k++)
                if (push(&all, &bv[b].v[k])) err = 1;
            free(bv[b].v);
        }
        free(bv);
    }
    free(G);
    if (err) { free(all.v); return -2; }
    *out = all.v;
    return all.n;
}

/*
 * PAM candidate list (the "search" kernel's output): ascending window starts p
 * in [begin, end) (clipped to 0 <= p <= len-L) whose strand-s reading passes the
 * pattern.  strand = '+' or '-'.  Returns the count and sets *out (free with
 * cof_oracle_free), or -1 on bad arguments, -2 on OOM.
 */
int64_t cof_oracle_pam_sites(const char *seq, int64_t len, int64_t begin, int64_t end,
                             const char *pattern_in, char strand, int64_t **out)
{
    int L = (int)strlen(pattern_in);
    *out = NULL;
    if (L < 1 || L > COF_ORACLE_MAX_L || (strand != '+' && strand != '-')) return -1;
    char P[COF_ORACLE_MAX_L + 1];
    for (int j = 0; j < L; j++) {
        P[j] = upper(pattern_in[j]);
        if (!is_iupac_code(P[j])) return -1;
    }
    int64_t lo = begin > 0 ? begin : 0, hi = len - L + 1;
    if (end < hi) hi = end;
    int64_t n = 0, cap = 1024;
    int64_t *v = (int64_t *)malloc((size_t)cap * sizeof(int64_t));
    if (!v) return -2;
    char S[COF_ORACLE_MAX_L + 1];
    for (int64_t p = lo; p < hi; p++) {
        window_reading(seq, p, L, strand, S);
        if (!pam_ok(S, P, L)) continue;
        if (n == cap) {
            cap *= 2;
            int64_t *nv = (int64_t *)realloc(v, (size_t)cap * sizeof(int64_t));
            if (!nv) { free(v); return -2; }
            v = nv;
        }
        v[n++] = p;
    }
    *out = v;
    return n;
}

void cof_oracle_free(void *p) { free(p); }

int32_t cof_oracle_hit_size(void) { return (int32_t)sizeof(oracle_hit); }

int32_t cof_oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
