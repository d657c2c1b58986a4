/*
 * oracle/oracle.c -- CPU ORACLE for the Jigsaw hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this library.  The product path (libjigsaw.so and the
 * Python binding) never links, imports or calls it; it shares no code, header,
 * table or constant generator with paper_conf_icpp_zhanglyfyllq24_b200/csrc.
 *
 * Plain, scalar, single-threaded C11.  Every function cites the passage of
 * /root/reference/PAPER.md (written P:NNN, the line number) or the DESIGN.md
 * reading (R-Qn, the ambiguity table of SURVEY.md §8c) it follows.
 *
 *   O1  orc_spmm           naive vector-sparse SpMM C = A.B, fp64 accumulate
 *   O2  orc_reorder_*      canonical reorder CR1 = multi-granularity reorder
 *                          (Alg. 1) + reorder-aware format
 *       orc_tile_reorder   Alg. 1 + reorder retry on ONE tile, generalised to
 *                          W columns / groups of G / at most Z nonzeros per group
 *                          (CR1 is W=16,G=4,Z=2; the Fig. 6 example is W=4,G=2,Z=1)
 *       orc_row_cluster    row order of the row-clustered panels (SURVEY §8(f) f2,
 *                          DESIGN.md R-Q27): CR1 is then applied to A[perm]
 *   (O3, the independent checker/decoder, is oracle/check.py: numpy, no call into O2.)
 *
 * Parity status: every function here is pinned by tests/test_oracle_*.py except
 * the tie-break choices CR1 makes where the paper is silent (R-Q8, R-Q10, R-Q11,
 * R-Q12): those are "parity unpinned" against the authors' unseen code -- only
 * validity and determinism are provable.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_PAD (-1)

/* ------------------------------------------------------------------------- */
/* IEEE-754 binary16 helpers                                                 */
/* ------------------------------------------------------------------------- */

/* Nonzero test (R-Q3): +0 and -0 are zero; every other pattern (NaN/Inf too)
 * is a nonzero.  Applied to the raw fp16 bits. */
static int nz16(uint16_t h) { return (h & 0x7FFFu) != 0; }

/* Exact binary16 -> double decode (sign, 5-bit exponent, 10-bit fraction). */
double orc_half_to_double(uint16_t h)
{
    int sign = (h >> 15) & 1;
    int expo = (h >> 10) & 0x1F;
    int frac = h & 0x3FF;
    double v;
    if (expo == 0) {
        v = (double)frac / 1024.0 / 16384.0;           /* subnormal: frac * 2^-24 */
    } else if (expo == 31) {
        v = frac ? __builtin_nan("") : __builtin_inf();
    } else {
        double m = 1.0 + (double)frac / 1024.0;
        int e = expo - 15;
        v = m;
        if (e > 0) { while (e--) v *= 2.0; }
        else       { while (e++) v *= 0.5; }
    }
    return sign ? -v : v;
}

/* ------------------------------------------------------------------------- */
/* O1: naive SpMM ("C = A x B", A sparse M x K, B dense K x N)  */
/* ------------------------------------------------------------------------- */

/* C[i][n]    = sum over k ascending with nz(A[i][k]) of A[i][k]*B[k][n]   (fp64)
 * Mabs[i][n] = sum over the same k of |A[i][k]|*|B[k][n]|               (fp64)
 * Only the rows listed in `rows` (nrows of them) are computed; rows == NULL
 * means all M rows.  Output row j of C/Mabs corresponds to rows[j].
 * A: M x K row-major fp16 bits; B: K x N row-major fp16 bits. */
int orc_spmm(const uint16_t *A, int64_t M, int64_t K,
             const uint16_t *B, int64_t N,
             const int64_t *rows, int64_t nrows,
             double *C, double *Mabs)
{
    if (!A || !B || !C || M <= 0 || K <= 0 || N <= 0) return 1;
    if (!rows) nrows = M;
    for (int64_t j = 0; j < nrows; ++j) {
        int64_t i = rows ? rows[j] : j;
        if (i < 0 || i >= M) return 2;
        double *c = C + j * N;
        double *mab = Mabs ? Mabs + j * N : NULL;
        for (int64_t n = 0; n < N; ++n) { c[n] = 0.0; if (mab) mab[n] = 0.0; }
        for (int64_t k = 0; k < K; ++k) {
            uint16_t a16 = A[i * K + k];
            if (!nz16(a16)) continue;
            double a = orc_half_to_double(a16);
            const uint16_t *brow = B + k * N;
            for (int64_t n = 0; n < N; ++n) {
                double b = orc_half_to_double(brow[n]);
                c[n] += a * b;
                if (mab) mab[n] += __builtin_fabs(a) * __builtin_fabs(b);
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Row masks: one P-bit mask per column of a panel (P <= 256, four 64-bit words)*/
/* ------------------------------------------------------------------------- */

#define MASK_WORDS 4
typedef struct { uint64_t w[MASK_WORDS]; } mask256;

static int mask_is_zero(mask256 m) { return (m.w[0] | m.w[1] | m.w[2] | m.w[3]) == 0; }

/* ------------------------------------------------------------------------- */
/* Alg. 1 + reorder retry on one tile                    */
/* ------------------------------------------------------------------------- */

typedef struct {
    int W, G, Z;                /* tile width, group size, max nonzeros per group and row */
    mask256 m[16];              /* per-slot row masks; PAD slots have mask 0 */
    int real[16];               /* 1 if the slot holds a real (non-PAD) column */
    unsigned char compat[1 << 16];   /* compat[S] for every G-subset S (bitmask of slots) */
    int nsub;                   /* number of G-subsets of W slots */
    uint32_t subs[1820 + 16];   /* the G-subsets, as bitmasks, in lexicographic order */
    int nby_lo[16];             /* the same subsets split by their smallest slot, */
    uint32_t by_lo[16][1820];   /* each list still in lexicographic order */
    int ncby_lo[16];            /* ... and only the compatible ones (rebuilt per attempt) */
    uint32_t cby_lo[16][1820];
    uint8_t dead[1 << 13];      /* dead[S]: bit set once "cover the rest of used-set S" failed */
    uint32_t chosen[16];        /* DFS stack of chosen groups */
} tile_ctx;

/* All G-subsets of {0..W-1} in lexicographic order of their sorted tuples. */
static void enum_subsets(tile_ctx *t)
{
    int idx[16];
    t->nsub = 0;
    for (int i = 0; i < t->G; ++i) idx[i] = i;
    for (;;) {
        uint32_t s = 0;
        for (int i = 0; i < t->G; ++i) s |= 1u << idx[i];
        t->subs[t->nsub++] = s;
        int i = t->G - 1;
        while (i >= 0 && idx[i] == t->W - t->G + i) --i;
        if (i < 0) break;
        ++idx[i];
        for (int j = i + 1; j < t->G; ++j) idx[j] = idx[j - 1] + 1;
    }
    for (int lo = 0; lo < 16; ++lo) t->nby_lo[lo] = 0;
    for (int k = 0; k < t->nsub; ++k) {
        int lo = __builtin_ctz(t->subs[k]);
        t->by_lo[lo][t->nby_lo[lo]++] = t->subs[k];
    }
}

/* Alg. 1 lines 1-8: a group of columns is compatible iff no row has more than
 * Z nonzeros among them ("if the number of non-zero elements in each row
 * does not exceed 2").  Counted with saturating bit-plane counters:
 * plane c[j] has a row bit set once that row has seen > j nonzeros. */
static int group_compatible(const tile_ctx *t, uint32_t s)
{
    for (int w = 0; w < MASK_WORDS; ++w) {
        uint64_t c[17] = {0};
        for (uint32_t rest = s; rest; rest &= rest - 1) {
            int j = __builtin_ctz(rest);
            uint64_t x = t->m[j].w[w];
            for (int q = t->Z; q >= 1; --q) c[q] |= c[q - 1] & x;
            c[0] |= x;
        }
        if (c[t->Z]) return 0;     /* some row has >= Z+1 nonzeros */
    }
    return 1;
}

/* Depth-first search for the lexicographically smallest partition (R-Q8):
 * always extend with a group containing the smallest uncovered slot, trying
 * candidate groups in lexicographic order.  `dead` remembers used-sets whose
 * remainder has no cover, so a failed subtree is not searched twice (this
 * changes only the running time, never which partition is found first). */
static int dfs(tile_ctx *t, uint32_t used, int depth)
{
    uint32_t full = (1u << t->W) - 1u;
    if (used == full) return 1;
    if (t->dead[used >> 3] & (1u << (used & 7))) return 0;
    int lo = __builtin_ctz(~used & full);
    for (int k = 0; k < t->ncby_lo[lo]; ++k) {
        uint32_t s = t->cby_lo[lo][k];
        if (s & used) continue;
        t->chosen[depth] = s;
        if (dfs(t, used | s, depth + 1)) return 1;
    }
    t->dead[used >> 3] |= (uint8_t)(1u << (used & 7));
    return 0;
}

/* TileReorder on one tile (R-Q8, R-Q11).
 *  masks  : W row masks (4 words each, row r of the panel is bit r%64 of word r/64)
 *  cols   : in/out, W column ids (ORC_PAD = -1); evicted slots become ORC_PAD
 *  perm   : out, W slot indices: the new column order g0 || g1 || ... (groups sorted)
 *  evicted: out, evicted column ids in eviction order; *nev their count
 * Returns 0 on success. */
int orc_tile_reorder(const uint64_t *masks, int W, int G, int Z,
                     int32_t *cols, uint8_t *perm, int32_t *evicted, int *nev)
{
    static tile_ctx tc;          /* single-threaded oracle: one static context */
    tile_ctx *t = &tc;
    if (W < 1 || W > 16 || G < 1 || G > W || W % G || Z < 0 || Z > G) return 1;
    long ncomb = 1;
    for (int i = 0; i < G; ++i) ncomb = ncomb * (W - i) / (i + 1);
    if (ncomb > 1820) return 1;                 /* subsets table capacity */
    t->W = W; t->G = G; t->Z = Z;
    enum_subsets(t);
    for (int j = 0; j < W; ++j) {
        t->real[j] = cols[j] != ORC_PAD;
        for (int w = 0; w < MASK_WORDS; ++w)
            t->m[j].w[w] = t->real[j] ? masks[MASK_WORDS * j + w] : 0;
    }
    *nev = 0;
    for (;;) {
        /* Alg. 1 lines 1-8: every compatible column group. */
        for (int k = 0; k < t->nsub; ++k)
            t->compat[t->subs[k]] = (unsigned char)group_compatible(t, t->subs[k]);
        /* freq[j] = number of compatible groups containing slot j. */
        long freq[16] = {0};
        int coverable = 1;
        for (int k = 0; k < t->nsub; ++k)
            if (t->compat[t->subs[k]])
                for (uint32_t rest = t->subs[k]; rest; rest &= rest - 1) ++freq[__builtin_ctz(rest)];
        for (int j = 0; j < W; ++j)
            if (freq[j] == 0) coverable = 0;   /* a slot no compatible group covers: no cover */
        for (int lo = 0; lo < 16; ++lo) {
            t->ncby_lo[lo] = 0;
            for (int k = 0; k < t->nby_lo[lo]; ++k)
                if (t->compat[t->by_lo[lo][k]]) t->cby_lo[lo][t->ncby_lo[lo]++] = t->by_lo[lo][k];
        }
        /* W/G disjoint groups hold at most (W/G) * (most real columns in one
         * compatible group) real columns: fewer than we have means no cover. */
        uint32_t realset = 0;
        int nreal = 0, hmax = 0;
        for (int j = 0; j < W; ++j) if (t->real[j]) { realset |= 1u << j; ++nreal; }
        for (int k = 0; k < t->nsub; ++k)
            if (t->compat[t->subs[k]]) {
                int h = __builtin_popcount(t->subs[k] & realset);
                if (h > hmax) hmax = h;
            }
        if (hmax * (W / G) < nreal) coverable = 0;
        /* Alg. 1 lines 9-17: a cover of the W columns by disjoint compatible groups. */
        memset(t->dead, 0, sizeof t->dead);
        if (coverable && dfs(t, 0u, 0)) {
            int o = 0;
            for (int g = 0; g < W / G; ++g)
                for (int j = 0; j < W; ++j)
                    if (t->chosen[g] & (1u << j)) perm[o++] = (uint8_t)j;
            return 0;
        }
        /* Reorder retry: the real column that appears least frequently
         * in all compatible groups is moved out and its slot becomes all-zero. */
        int best = -1;
        for (int j = 0; j < W; ++j)
            if (t->real[j] && (best < 0 || freq[j] < freq[best])) best = j;   /* ties: smallest slot */
        if (best < 0) return 2;   /* unreachable: an all-PAD tile always has a cover */
        evicted[(*nev)++] = cols[best];
        cols[best] = ORC_PAD;
        t->real[best] = 0;
        for (int w = 0; w < MASK_WORDS; ++w) t->m[best].w[w] = 0;
    }
}

/* ------------------------------------------------------------------------- */
/* O2: CR1 over a whole matrix                                               */
/* ------------------------------------------------------------------------- */

typedef struct {
    int64_t M, K;
    int P, mode, npanels;
    int64_t *T, *D;               /* per panel: 2:4 tiles, dense residual tiles */
    int64_t ntiles, ndtiles, cap, dcap;
    int32_t *col_idx;             /* [ntiles][16] */
    uint8_t *perm;                /* [ntiles][16] */
    uint16_t *vals;               /* [ntiles][P][8] */
    uint16_t *meta;               /* [ntiles][P] */
    uint8_t *kind;                /* [ntiles] 0 = MAIN, 1 = OVERFLOW (label only) */
    uint8_t *nevict;              /* [ntiles] evictions performed in that tile */
    int32_t *rcol;                /* [ndtiles][16]  DENSE mode residual columns */
    uint16_t *dvals;              /* [ndtiles][P][16] DENSE mode residual values */
} orc_format;

static int grow(orc_format *f, int64_t need)
{
    if (need <= f->cap) return 0;
    int64_t cap = f->cap ? f->cap : 64;
    while (cap < need) cap *= 2;
    int P = f->P;
    f->col_idx = realloc(f->col_idx, (size_t)cap * 16 * sizeof(int32_t));
    f->perm    = realloc(f->perm, (size_t)cap * 16);
    f->vals    = realloc(f->vals, (size_t)cap * P * 8 * sizeof(uint16_t));
    f->meta    = realloc(f->meta, (size_t)cap * P * sizeof(uint16_t));
    f->kind    = realloc(f->kind, (size_t)cap);
    f->nevict  = realloc(f->nevict, (size_t)cap);
    if (!f->col_idx || !f->perm || !f->vals || !f->meta || !f->kind || !f->nevict) return 1;
    f->cap = cap;
    return 0;
}

static int dgrow(orc_format *f, int64_t need)
{
    if (need <= f->dcap) return 0;
    int64_t cap = f->dcap ? f->dcap : 16;
    while (cap < need) cap *= 2;
    f->rcol  = realloc(f->rcol, (size_t)cap * 16 * sizeof(int32_t));
    f->dvals = realloc(f->dvals, (size_t)cap * f->P * 16 * sizeof(uint16_t));
    if (!f->rcol || !f->dvals) return 1;
    f->dcap = cap;
    return 0;
}

/* A element (r, c) of the matrix; rows >= M (last panel) and PAD read as zero (R-Q20). */
static uint16_t a_at(const uint16_t *A, int64_t M, int64_t K, int64_t r, int32_t c)
{
    if (c == ORC_PAD || r >= M) return 0;
    return A[r * K + c];
}

/* Reorder-aware compression of one tile (P:96 metadata; R-Q15, R-Q16):
 * per row r and group q, positions i = 0..3 map to columns col_idx[perm[4q+i]];
 * keep = the nonzero positions plus the smallest zero positions up to two,
 * sorted (i0 < i1); vals = the kept fp16 bits (0 for a kept zero);
 * meta nibble q = i0 + 4*i1. */
static void compress_tile(orc_format *f, const uint16_t *A, int64_t row0, int64_t t)
{
    const int32_t *ci = f->col_idx + t * 16;
    const uint8_t *pm = f->perm + t * 16;
    for (int r = 0; r < f->P; ++r) {
        uint16_t meta = 0;
        uint16_t *v = f->vals + ((size_t)t * f->P + r) * 8;
        for (int q = 0; q < 4; ++q) {
            int keep[2], nk = 0;
            uint16_t bits[4];
            for (int i = 0; i < 4; ++i) bits[i] = a_at(A, f->M, f->K, row0 + r, ci[pm[4 * q + i]]);
            for (int i = 0; i < 4 && nk < 2; ++i) if (nz16(bits[i])) keep[nk++] = i;
            for (int i = 0; i < 4 && nk < 2; ++i) {
                if (nz16(bits[i])) continue;
                int dup = 0;
                for (int k = 0; k < nk; ++k) dup |= keep[k] == i;
                if (!dup) keep[nk++] = i;
            }
            if (keep[0] > keep[1]) { int x = keep[0]; keep[0] = keep[1]; keep[1] = x; }
            for (int k = 0; k < 2; ++k)
                v[2 * q + k] = nz16(bits[keep[k]]) ? bits[keep[k]] : 0;
            meta |= (uint16_t)((keep[0] + 4 * keep[1]) << (4 * q));
        }
        f->meta[(size_t)t * f->P + r] = meta;
    }
}

/* CR1 over panels [p0, p1) of A (M x K fp16 bits, row-major).
 *   P    : panel rows (1..256)                         (R-Q5, R-Q6)
 *   mode : 0 = SPTC (paper: evicted columns re-queued)
 *          1 = DENSE (evicted columns -> dense residual tail; R-Q12)
 * Returns an opaque format or NULL. */
void *orc_reorder_range(const uint16_t *A, int64_t M, int64_t K, int P, int mode,
                        int p0, int p1)
{
    if (!A || M <= 0 || K <= 0 || P < 1 || P > 256 || (mode != 0 && mode != 1)) return NULL;
    int npan = (int)((M + P - 1) / P);
    if (p0 < 0 || p1 > npan || p0 > p1) return NULL;
    orc_format *f = calloc(1, sizeof(orc_format));
    if (!f) return NULL;
    f->M = M; f->K = K; f->P = P; f->mode = mode; f->npanels = p1 - p0;
    f->T = calloc((size_t)(p1 - p0) + 1, sizeof(int64_t));
    f->D = calloc((size_t)(p1 - p0) + 1, sizeof(int64_t));
    mask256 *cm = malloc((size_t)K * sizeof(mask256));
    int32_t *queue = malloc((size_t)(K + 16) * 2 * sizeof(int32_t) + 64);
    int32_t *resid = malloc((size_t)(K + 16) * sizeof(int32_t) + 64);
    if (!f->T || !f->D || !cm || !queue || !resid) { free(cm); free(queue); free(resid); return NULL; }

    for (int p = p0; p < p1; ++p) {
        int64_t row0 = (int64_t)p * P;
        /* BLOCK_TILE granularity: per-column row masks, then S_p =
         * the columns with any nonzero, in ascending order (R-Q4, Fig. 6). */
        int64_t head = 0, tail = 0;
        for (int64_t c = 0; c < K; ++c) {
            mask256 m = {{0, 0, 0, 0}};
            for (int r = 0; r < P; ++r)
                if (nz16(a_at(A, M, K, row0 + r, (int32_t)c))) m.w[r / 64] |= 1ull << (r % 64);
            cm[c] = m;
            if (!mask_is_zero(m)) queue[tail++] = (int32_t)c;
        }
        int64_t nS = tail, nmain = (nS + 15) / 16, nres = 0;
        int64_t tp = 0;
        /* MMA_TILE granularity: pop up to 16 columns per tile. */
        while (head < tail) {
            int32_t cols[16];
            uint64_t mk[16 * MASK_WORDS];
            for (int j = 0; j < 16; ++j) {
                cols[j] = head < tail ? queue[head++] : ORC_PAD;
                mask256 m = cols[j] == ORC_PAD ? (mask256){{0, 0, 0, 0}} : cm[cols[j]];
                for (int w = 0; w < MASK_WORDS; ++w) mk[MASK_WORDS * j + w] = m.w[w];
            }
            uint8_t perm[16]; int32_t ev[16]; int nev = 0;
            if (orc_tile_reorder(mk, 16, 4, 2, cols, perm, ev, &nev)) return NULL;
            if (grow(f, f->ntiles + 1)) return NULL;
            int64_t t = f->ntiles++;
            memcpy(f->col_idx + t * 16, cols, sizeof cols);
            memcpy(f->perm + t * 16, perm, sizeof perm);
            f->kind[t] = tp < nmain ? 0 : 1;
            f->nevict[t] = (uint8_t)nev;
            compress_tile(f, A, row0, t);
            ++tp;
            for (int e = 0; e < nev; ++e) {
                if (mode == 0) queue[tail++] = ev[e];     /* back of the panel FIFO */
                else           resid[nres++] = ev[e];     /* dense residual list R_p */
            }
        }
        f->T[p - p0] = tp;
        /* DENSE mode: R_p in chunks of 16, dense fp16 tiles, identity order. */
        int64_t dp = 0;
        for (int64_t s = 0; s < nres; s += 16, ++dp) {
            if (dgrow(f, f->ndtiles + 1)) return NULL;
            int64_t d = f->ndtiles++;
            for (int j = 0; j < 16; ++j) f->rcol[d * 16 + j] = s + j < nres ? resid[s + j] : ORC_PAD;
            for (int r = 0; r < P; ++r)
                for (int j = 0; j < 16; ++j) {
                    uint16_t b = a_at(A, M, K, row0 + r, f->rcol[d * 16 + j]);
                    f->dvals[((size_t)d * P + r) * 16 + j] = nz16(b) ? b : 0;
                }
        }
        f->D[p - p0] = dp;
    }
    free(cm); free(queue); free(resid);
    return f;
}

void *orc_reorder(const uint16_t *A, int64_t M, int64_t K, int P, int mode)
{
    int npan = (int)((M + P - 1) / (P > 0 ? P : 1));
    return orc_reorder_range(A, M, K, P, mode, 0, npan);
}

/* Accessors: sizes, then copies into caller-allocated buffers. */
void orc_format_sizes(const void *h, int64_t *out /* [4]: npanels, ntiles, ndtiles, P */)
{
    const orc_format *f = h;
    out[0] = f->npanels; out[1] = f->ntiles; out[2] = f->ndtiles; out[3] = f->P;
}

void orc_format_copy(const void *h, int64_t *T, int64_t *D, int32_t *col_idx, uint8_t *perm,
                     uint16_t *vals, uint16_t *meta, uint8_t *kind, uint8_t *nevict,
                     int32_t *rcol, uint16_t *dvals)
{
    const orc_format *f = h;
    int64_t n = f->ntiles, d = f->ndtiles; int P = f->P;
    memcpy(T, f->T, (size_t)f->npanels * sizeof(int64_t));
    memcpy(D, f->D, (size_t)f->npanels * sizeof(int64_t));
    if (n) {
        memcpy(col_idx, f->col_idx, (size_t)n * 16 * sizeof(int32_t));
        memcpy(perm, f->perm, (size_t)n * 16);
        memcpy(vals, f->vals, (size_t)n * P * 8 * sizeof(uint16_t));
        memcpy(meta, f->meta, (size_t)n * P * sizeof(uint16_t));
        memcpy(kind, f->kind, (size_t)n);
        memcpy(nevict, f->nevict, (size_t)n);
    }
    if (d) {
        memcpy(rcol, f->rcol, (size_t)d * 16 * sizeof(int32_t));
        memcpy(dvals, f->dvals, (size_t)d * P * 16 * sizeof(uint16_t));
    }
}

void orc_format_free(void *h)
{
    orc_format *f = h;
    if (!f) return;
    free(f->T); free(f->D); free(f->col_idx); free(f->perm); free(f->vals);
    free(f->meta); free(f->kind); free(f->nevict); free(f->rcol); free(f->dvals);
    free(f);
}

/* ------------------------------------------------------------------------- */
/* Row-clustered panels (DESIGN.md R-Q27, not in the paper:  */
/* the B200 analogue of its small BLOCK_TILE)                   */
/* ------------------------------------------------------------------------- */

/* perm[i] = the i-th row of A in order of decreasing nonzero count (nz16),
 * rows with equal counts in ascending index order.  Written as the definition:
 * for every count from K down to 0, the rows with that count, scanned in order. */
int orc_row_cluster(const uint16_t *A, int64_t M, int64_t K, int32_t *perm)
{
    int64_t *cnt = (int64_t *)malloc(sizeof(int64_t) * (size_t)(M > 0 ? M : 1));
    if (!cnt) return 1;
    for (int64_t r = 0; r < M; ++r) {
        cnt[r] = 0;
        for (int64_t k = 0; k < K; ++k) cnt[r] += nz16(A[r * K + k]);
    }
    int64_t i = 0;
    for (int64_t c = K; c >= 0; --c)
        for (int64_t r = 0; r < M; ++r)
            if (cnt[r] == c) perm[i++] = (int32_t)r;
    free(cnt);
    return i == M ? 0 : 2;
}
