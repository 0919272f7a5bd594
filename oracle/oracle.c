/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle for TileSpMV
 *             (Niu, Lu, Dong, Jin, Liu, Tan, IPDPS 2021; /root/reference/PAPER.md).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_niuldj0t21_b200/csrc/); neither side includes the other.
 *
 * Citations "P:n" are lines of PAPER.md; "R<k>" are the readings listed in
 * DESIGN.md §"Readings of the paper" (SURVEY.md §8c C3 #k).
 *
 * Contents
 *   oracle_spmv_f64    Alg. 1 word for word in double: the plain
 *                      fp64 row loop, the CPU baseline bench.py times
 *                      (BASELINE.md D5 item 1); correctness uses
 *                      oracle_spmv_rows
 *   oracle_spmv_rows   Alg. 1: y_i = sum_j a_ij * x_j, every row
 *                      independent, accumulated in x87 long double and rounded
 *                      once; also sum_j |a_ij * x_j| for the tolerance test.
 *   oracle_select      the TileSpMV_ADPT format rules.
 *   oracle_select_bytes  the optional B200 byte-cost selection (SURVEY
 *                      §8(f) f4; NOT the paper's rule): fewest payload bytes.
 *   oracle_hyb_width   the HYB ELL-width scan.
 *   oracle_tile        two-level tiled storage with the
 *                      DeferredCOO extraction, laid out in the
 *                      canonical byte layout of DESIGN.md §"Canonical layout".
 *   oracle_decode      inverse of oracle_tile (round-trip pin).
 *
 * Parity status (DESIGN.md §"Oracle pins"): every function here is pinned by
 * tests/test_oracle_*.py against closed forms, brute force or hand-built
 * cases; none is "parity unpinned".
 */
#include <float.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

_Static_assert(LDBL_MANT_DIG == 64, "oracle needs x87 80-bit long double");

/* tile formats, numbered in the order the paper lists them */
enum { O_CSR = 0, O_COO = 1, O_ELL = 2, O_HYB = 3, O_DNS = 4, O_DNSROW = 5, O_DNSCOL = 6 };
/* the three TileSpMV methods of P:177 (+ the size switch of P:235) */
enum { O_MODE_ADPT = 0, O_MODE_DEFERRED = 1, O_MODE_AUTO = 2, O_MODE_FORCE_CSR = 3, O_MODE_BYTES = 4 };

#define TILE 16 /* "the size is always 16 by 16" */

/* ------------------------------------------------------------------------ */
/* Alg. 1                                                         */
/* ------------------------------------------------------------------------ */

/* For each requested row i (all rows if rows == NULL):
 *   y_i    <- 0;  for each nonzero a_ij in row i: y_i <- y_i + a_ij * x_j
 *   absy_i <- sum_j |a_ij * x_j|
 * The accumulator is long double (64-bit mantissa): the error is at most
 * (k+1) * 2^-63 * absy_i before the single final rounding to double, far
 * below the 1e-12 * absy_i acceptance bound. */
int oracle_spmv_rows(int64_t m, const int32_t *rowptr, const int32_t *colidx,
                     const double *val, const double *x, const int64_t *rows,
                     int64_t nrows, double *y, double *absy)
{
    if (rows == NULL) nrows = m;
    for (int64_t q = 0; q < nrows; ++q) {
        int64_t i = rows ? rows[q] : q;
        if (i < 0 || i >= m) return -1;
        long double yi = 0.0L;
        long double ai = 0.0L;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
            long double p = (long double)val[k] * (long double)x[colidx[k]];
            yi += p;
            ai += p < 0 ? -p : p;
        }
        y[q] = (double)yi;
        if (absy) absy[q] = (double)ai;
    }
    return 0;
}

/* Alg. 1 as printed, in double: y_i <- 0, then y_i <- y_i +
 * a_ij * x_j in entry order, each product and sum rounded to double (gcc
 * -O2 without -ffast-math and without FMA contraction keeps that order). */
void oracle_spmv_f64(int64_t m, const int32_t *rowptr, const int32_t *colidx,
                     const double *val, const double *x, double *y)
{
    for (int64_t i = 0; i < m; ++i) {
        double yi = 0.0;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) yi = yi + val[k] * x[colidx[k]];
        y[i] = yi;
    }
}

/* ------------------------------------------------------------------------ */
/* Format selection, TileSpMV_ADPT                              */
/* ------------------------------------------------------------------------ */

static int popc16(unsigned v) { int c = 0; while (v) { c += v & 1u; v >>= 1; } return c; }

/* masks[r] bit c set <=> entry (r, c) of the 16x16 tile is stored.
 * Returns the format, writes the auxiliary byte (ELL/HYB width, number of
 * dense rows/cols, else 0).  Rules, in the text order of P:181-197 (R7):
 *   1. COO    : nnz < 12 (the "not evenly" clause is implied, R4)
 *   2. Dns    : nnz >= 128 (R5)
 *   3. DnsRow : every row holds 0 or 16 entries (R6)
 *   4. DnsCol : every column holds 0 or 16 entries (R6)
 *   5. variation = std / mean of the 16 row lengths (population std, R8):
 *      ELL if variation <= te = 0.2; HYB if variation > th = 1.0; else CSR
 *      (R9).  Evaluated exactly in integers: with
 *      D = sum_r (16*len_r - nnz)^2, variation^2 = D / (16 * nnz^2).       */
int oracle_hyb_width(const int32_t lens[16]);

int oracle_select(const uint16_t masks[16], int32_t force_csr, int32_t *aux)
{
    int32_t lens[16];
    int64_t nnz = 0;
    int32_t colcnt[16] = {0};
    for (int r = 0; r < TILE; ++r) {
        lens[r] = popc16(masks[r]);
        nnz += lens[r];
        for (int c = 0; c < TILE; ++c)
            if ((masks[r] >> c) & 1u) colcnt[c]++;
    }
    *aux = 0;
    if (force_csr) return O_CSR; /* TileSpMV_CSR */
    if (nnz < 12) return O_COO;
    if (nnz >= 128) return O_DNS;
    int rows_full = 1, cols_full = 1, nr = 0, nc = 0;
    for (int r = 0; r < TILE; ++r) {
        if (lens[r] != 0 && lens[r] != TILE) rows_full = 0;
        if (lens[r] == TILE) nr++;
    }
    for (int c = 0; c < TILE; ++c) {
        if (colcnt[c] != 0 && colcnt[c] != TILE) cols_full = 0;
        if (colcnt[c] == TILE) nc++;
    }
    if (rows_full) { *aux = nr; return O_DNSROW; }
    if (cols_full) { *aux = nc; return O_DNSCOL; }
    /* mean = nnz/16, var = sum (len - mean)^2 / 16 = D / 4096,
     * variation^2 = var / mean^2 = D / (16 nnz^2)                           */
    int64_t D = 0;
    for (int r = 0; r < TILE; ++r) {
        int64_t d = 16 * (int64_t)lens[r] - nnz;
        D += d * d;
    }
    /* variation <= 0.2  <=>  D/(16 nnz^2) <= 1/25  <=>  25 D <= 16 nnz^2 */
    if (25 * D <= 16 * nnz * nnz) {
        int32_t w = 0;
        for (int r = 0; r < TILE; ++r) if (lens[r] > w) w = lens[r];
        *aux = w; /* tilewidth = maximum row length */
        return O_ELL;
    }
    /* variation > 1.0  <=>  D > 16 nnz^2 */
    if (D > 16 * nnz * nnz) {
        *aux = oracle_hyb_width(lens);
        return O_HYB;
    }
    return O_CSR;
}

/* B200 byte-cost selection (TILESPMV_MODE_BYTES; not the
 * paper's rule, so no parity with its format statistics is claimed): the
 * format whose payload, by the sizes of DESIGN.md §4 rounded up to 16 bytes,
 * is smallest among the formats able to hold the tile:
 *   CSR     8 nnz + 16 + ceil(nnz / 2)       any tile
 *   COO     9 nnz                            any tile
 *   ELL     136 * (max row length)           every row non-empty (R26: a pad
 *                                            must be told from an entry)
 *   HYB     136 w + 9 (nnz - 16 w), w = oracle_hyb_width (R11)   any tile
 *   Dns     2048                             any tile
 *   DnsRow  129 * (full rows)                every row 0 or 16 entries (R6)
 *   DnsCol  129 * (full columns)             every column 0 or 16 entries
 * Ties go to the lowest format code (P:96 order).  aux as oracle_select.   */
int oracle_select_bytes(const uint16_t masks[16], int32_t *aux)
{
    int32_t lens[16];
    int64_t nnz = 0;
    int32_t colcnt[16] = {0};
    for (int r = 0; r < TILE; ++r) {
        lens[r] = popc16(masks[r]);
        nnz += lens[r];
        for (int c = 0; c < TILE; ++c)
            if ((masks[r] >> c) & 1u) colcnt[c]++;
    }
    int32_t maxlen = 0, minlen = TILE, nr = 0, nc = 0, rows_full = 1, cols_full = 1;
    for (int r = 0; r < TILE; ++r) {
        if (lens[r] > maxlen) maxlen = lens[r];
        if (lens[r] < minlen) minlen = lens[r];
        if (lens[r] != 0 && lens[r] != TILE) rows_full = 0;
        if (lens[r] == TILE) nr++;
    }
    for (int c = 0; c < TILE; ++c) {
        if (colcnt[c] != 0 && colcnt[c] != TILE) cols_full = 0;
        if (colcnt[c] == TILE) nc++;
    }
    int32_t hw = oracle_hyb_width(lens);
    int64_t size[7];
    int32_t faux[7] = {0, 0, maxlen, hw, 0, nr, nc};
    int eligible[7] = {1, 1, minlen >= 1, 1, 1, rows_full, cols_full};
    size[O_CSR] = 8 * nnz + 16 + (nnz + 1) / 2;
    size[O_COO] = 9 * nnz;
    size[O_ELL] = 136 * (int64_t)maxlen;
    size[O_HYB] = 136 * (int64_t)hw + 9 * (nnz - 16 * (int64_t)hw);
    size[O_DNS] = 2048;
    size[O_DNSROW] = 129 * (int64_t)nr;
    size[O_DNSCOL] = 129 * (int64_t)nc;
    int best = -1;
    int64_t best_size = 0;
    for (int f = 0; f < 7; ++f) {
        if (!eligible[f]) continue;
        int64_t sz = (size[f] + 15) / 16 * 16;
        if (best < 0 || sz < best_size) { best = f; best_size = sz; }
    }
    *aux = faux[best];
    return best;
}

/* "gradually calculate the least memory space by setting the ELL width
 * from the maximum to zero until the smallest memory space is found".
 * Memory of a width-w HYB tile (R11): 16*w ELL slots of value + 4-bit column
 * (8.5 B) plus one value + packed row/col byte (9 B) per entry beyond
 * the first w of its row.  Scanned from max down to 0; the first minimum
 * found wins (ties keep the larger width, as Fig. 3's HYB tile does).
 * Costs are doubled to stay in integers.                                    */
int oracle_hyb_width(const int32_t lens[16])
{
    int32_t maxlen = 0;
    for (int r = 0; r < TILE; ++r) if (lens[r] > maxlen) maxlen = lens[r];
    int64_t best_mem = -1;
    int32_t best_w = maxlen;
    for (int32_t w = maxlen; w >= 0; --w) {
        int64_t mem2 = (int64_t)TILE * w * 17; /* 2 * 8.5 B per ELL slot */
        for (int r = 0; r < TILE; ++r)
            if (lens[r] > w) mem2 += (int64_t)(lens[r] - w) * 18; /* 2 * 9 B */
        if (best_mem < 0 || mem2 < best_mem) { best_mem = mem2; best_w = w; }
    }
    return best_w;
}

/* ------------------------------------------------------------------------ */
/* Reference tiler                                 */
/* ------------------------------------------------------------------------ */

typedef struct {
    int64_t m, n, nnz, tilem, tilen;
    int32_t mode; /* resolved: ADPT, DEFERRED or FORCE_CSR */
    int64_t numtile;
    int32_t *tilePtr;    /* tilem + 1 */
    int32_t *tileColIdx; /* numtile */
    int32_t *tileNnz;    /* numtile + 1, prefix of held nonzeros */
    uint8_t *tileFmt;    /* numtile */
    uint8_t *tileAux;    /* numtile */
    uint32_t *tileOff;   /* numtile + 1, payload offsets in 16-byte units */
    uint8_t *payload;
    int64_t payload_bytes;
    int32_t *remRowPtr; /* m + 1 */
    int32_t *remCol;
    double *remVal;
    int64_t rem_nnz;
    int64_t sel_tiles[7], sel_nnz[7];   /* formats chosen by ADPT rules */
    int64_t kept_tiles[7], kept_nnz[7]; /* tiles actually stored */
} oracle_tiling;

typedef struct { int32_t J, r, c; int64_t k; } ent_t;

static int ent_cmp(const void *a, const void *b)
{
    const ent_t *x = a, *y = b;
    if (x->J != y->J) return x->J < y->J ? -1 : 1;
    if (x->r != y->r) return x->r < y->r ? -1 : 1;
    if (x->c != y->c) return x->c < y->c ? -1 : 1;
    return 0;
}

typedef struct { uint8_t *p; int64_t len, cap; } bytes_t;

static int bytes_reserve(bytes_t *b, int64_t extra)
{
    if (b->len + extra <= b->cap) return 0;
    int64_t cap = b->cap ? b->cap : 4096;
    while (cap < b->len + extra) cap *= 2;
    uint8_t *p = realloc(b->p, (size_t)cap);
    if (!p) return -1;
    b->p = p;
    b->cap = cap;
    return 0;
}

static void put_f64(uint8_t *dst, double v) { memcpy(dst, &v, 8); } /* bit copy */

static void put_nibble(uint8_t *base, int64_t idx, int v)
{ /* entry idx in byte idx/2, low nibble first (R12, R14) */
    if (idx % 2 == 0) base[idx / 2] |= (uint8_t)(v & 15);
    else base[idx / 2] |= (uint8_t)((v & 15) << 4);
}

void oracle_tiling_free(oracle_tiling *t)
{
    if (!t) return;
    free(t->tilePtr); free(t->tileColIdx); free(t->tileNnz); free(t->tileFmt);
    free(t->tileAux); free(t->tileOff); free(t->payload); free(t->remRowPtr);
    free(t->remCol); free(t->remVal);
    free(t);
}

/* mode: ADPT, DEFERRED, AUTO (DEFERRED iff nnz >= 1.8e6, R18), FORCE_CSR, or
 * BYTES (oracle_select_bytes, no extraction).
 * Returns NULL on allocation failure or non-canonical input.               */
oracle_tiling *oracle_tile(int64_t m, int64_t n, const int32_t *rowptr,
                           const int32_t *colidx, const double *val, int32_t mode)
{
    oracle_tiling *T = calloc(1, sizeof *T);
    if (!T) return NULL;
    int64_t nnz = m > 0 ? rowptr[m] : 0;
    if (mode == O_MODE_AUTO) mode = nnz >= 1800000 ? O_MODE_DEFERRED : O_MODE_ADPT;
    T->m = m; T->n = n; T->nnz = nnz; T->mode = mode;
    T->tilem = (m + TILE - 1) / TILE; /* edge tiles are partial (R1) */
    T->tilen = (n + TILE - 1) / TILE;

    /* canonical input check (step 1 of DESIGN.md §"Reference tiler") */
    if (m > 0 && rowptr[0] != 0) goto fail;
    for (int64_t i = 0; i < m; ++i) {
        if (rowptr[i + 1] < rowptr[i]) goto fail;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
            if (colidx[k] < 0 || colidx[k] >= n) goto fail;
            if (k > rowptr[i] && colidx[k] <= colidx[k - 1]) goto fail;
        }
    }

    int deferred = (mode == O_MODE_DEFERRED);
    int force_csr = (mode == O_MODE_FORCE_CSR);
    uint8_t *extracted = calloc((size_t)(nnz > 0 ? nnz : 1), 1);
    T->tilePtr = calloc((size_t)(T->tilem + 1), sizeof(int32_t));
    int64_t cap_tiles = 1024, ntile = 0;
    T->tileColIdx = malloc((size_t)cap_tiles * sizeof(int32_t));
    T->tileFmt = malloc((size_t)cap_tiles);
    T->tileAux = malloc((size_t)cap_tiles);
    int32_t *held = malloc((size_t)cap_tiles * sizeof(int32_t));
    int64_t *offs = malloc((size_t)cap_tiles * sizeof(int64_t));
    bytes_t pay = {0};
    ent_t *ents = NULL;
    int64_t ents_cap = 0;
    if (!extracted || !T->tilePtr || !T->tileColIdx || !T->tileFmt || !T->tileAux ||
        !held || !offs) goto fail_free;

    for (int64_t I = 0; I < T->tilem; ++I) {
        /* step 2: bucket the entries of tile row I into tiles (I, J = col/16) */
        int64_t r0 = I * TILE, r1 = r0 + TILE < m ? r0 + TILE : m;
        int64_t cnt = rowptr[r1] - rowptr[r0];
        if (cnt > ents_cap) {
            ents_cap = cnt * 2;
            ent_t *e2 = realloc(ents, (size_t)ents_cap * sizeof(ent_t));
            if (!e2) goto fail_free;
            ents = e2;
        }
        int64_t q = 0;
        for (int64_t i = r0; i < r1; ++i)
            for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
                ents[q].J = colidx[k] / TILE;
                ents[q].r = (int32_t)(i - r0);
                ents[q].c = colidx[k] % TILE;
                ents[q].k = k;
                q++;
            }
        /* step 3-4: tiles ordered by J, entries row-major inside a tile (R3) */
        qsort(ents, (size_t)cnt, sizeof(ent_t), ent_cmp);
        T->tilePtr[I] = (int32_t)ntile;
        for (int64_t a = 0; a < cnt;) {
            int64_t b = a;
            while (b < cnt && ents[b].J == ents[a].J) b++;
            const ent_t *e = ents + a;
            int64_t nt = b - a;
            uint16_t masks[16] = {0};
            int32_t lens[16] = {0};
            for (int64_t p = 0; p < nt; ++p) {
                masks[e[p].r] |= (uint16_t)(1u << e[p].c);
                lens[e[p].r]++;
            }
            /* step 5: select the format */
            int32_t aux;
            int fmt = mode == O_MODE_BYTES ? oracle_select_bytes(masks, &aux) : oracle_select(masks, force_csr, &aux);
            T->sel_tiles[fmt]++;
            T->sel_nnz[fmt] += nt;
            /* step 7: DeferredCOO extracts COO tiles and HYB COO parts */
            int store_fmt = fmt;
            int32_t store_aux = aux, store_nnz = (int32_t)nt;
            if (deferred && fmt == O_COO) {
                for (int64_t p = 0; p < nt; ++p) extracted[e[p].k] = 1;
                a = b;
                continue; /* tile removed (R17) */
            }
            if (deferred && fmt == O_HYB) {
                /* entries beyond the first w of their row are the COO part */
                int32_t rank[16] = {0};
                for (int64_t p = 0; p < nt; ++p) {
                    if (rank[e[p].r] >= aux) extracted[e[p].k] = 1;
                    rank[e[p].r]++;
                }
                if (aux == 0) { a = b; continue; } /* nothing left in the tile */
                store_fmt = O_ELL;  /* the residual is an ELL(w) tile, no pads */
                store_nnz = TILE * aux;
            }
            /* step 8: pack the level-2 payload (C2) */
            int64_t sz;
            switch (store_fmt) {
            case O_CSR: sz = 8 * nt + 16 + (nt + 1) / 2; break;
            case O_COO: sz = 9 * nt; break;
            case O_ELL: sz = 136 * (int64_t)store_aux; break;
            case O_HYB: sz = 136 * (int64_t)store_aux + 9 * (nt - TILE * (int64_t)store_aux); break;
            case O_DNS: sz = 2048; break;
            default: sz = 129 * (int64_t)store_aux; break; /* DnsRow / DnsCol */
            }
            int64_t sz16 = (sz + 15) / 16 * 16;
            if (bytes_reserve(&pay, sz16)) goto fail_free;
            uint8_t *P = pay.p + pay.len;
            memset(P, 0, (size_t)sz16); /* padding and empty slots are +0.0 */
            switch (store_fmt) {
            case O_CSR: { /* csrVal row-major, csrRowPtr[16] u8, 4-bit cols */
                for (int64_t p = 0; p < nt; ++p) put_f64(P + 8 * p, val[e[p].k]);
                uint8_t *rp = P + 8 * nt;
                int32_t acc = 0;
                for (int r = 0; r < TILE; ++r) { rp[r] = (uint8_t)acc; acc += lens[r]; }
                for (int64_t p = 0; p < nt; ++p) put_nibble(P + 8 * nt + 16, p, e[p].c);
                break;
            }
            case O_COO: /* cooVal, packed (row << 4 | col) (R13) */
                for (int64_t p = 0; p < nt; ++p) {
                    put_f64(P + 8 * p, val[e[p].k]);
                    P[8 * nt + p] = (uint8_t)((e[p].r << 4) | e[p].c);
                }
                break;
            case O_ELL: { /* column-major slots k*16 + r */
                int32_t w = store_aux, rank[16] = {0};
                for (int64_t p = 0; p < nt; ++p) {
                    int32_t kk = rank[e[p].r]++;
                    if (kk >= w) continue; /* only for ex-HYB tiles: extracted */
                    int64_t s = (int64_t)kk * TILE + e[p].r;
                    put_f64(P + 8 * s, val[e[p].k]);
                    put_nibble(P + 128 * (int64_t)w, s, e[p].c);
                }
                break;
            }
            case O_HYB: { /* ELL part (w) + COO part, ADPT mode only */
                int32_t w = store_aux, rank[16] = {0};
                int64_t kc = nt - TILE * (int64_t)w, qc = 0;
                uint8_t *ellv = P, *coov = P + 128 * (int64_t)w;
                uint8_t *elli = coov + 8 * kc, *cooi = elli + 8 * (int64_t)w;
                for (int64_t p = 0; p < nt; ++p) {
                    int32_t kk = rank[e[p].r]++;
                    if (kk < w) {
                        int64_t s = (int64_t)kk * TILE + e[p].r;
                        put_f64(ellv + 8 * s, val[e[p].k]);
                        put_nibble(elli, s, e[p].c);
                    } else {
                        put_f64(coov + 8 * qc, val[e[p].k]);
                        cooi[qc] = (uint8_t)((e[p].r << 4) | e[p].c);
                        qc++;
                    }
                }
                break;
            }
            case O_DNS: /* dnsVal column-major */
                for (int64_t p = 0; p < nt; ++p)
                    put_f64(P + 8 * ((int64_t)e[p].c * TILE + e[p].r), val[e[p].k]);
                break;
            case O_DNSROW: { /* values of full rows, rowid (R15) */
                int qmap[16], qn = 0;
                for (int r = 0; r < TILE; ++r) qmap[r] = lens[r] == TILE ? qn++ : -1;
                for (int64_t p = 0; p < nt; ++p)
                    put_f64(P + 8 * ((int64_t)qmap[e[p].r] * TILE + e[p].c), val[e[p].k]);
                for (int r = 0; r < TILE; ++r)
                    if (qmap[r] >= 0) P[128 * (int64_t)qn + qmap[r]] = (uint8_t)r;
                break;
            }
            case O_DNSCOL: { /* values of full columns, colid (R15) */
                int qmap[16], qn = 0;
                for (int c = 0; c < TILE; ++c) qmap[c] = ((masks[0] >> c) & 1u) ? qn++ : -1;
                for (int64_t p = 0; p < nt; ++p)
                    put_f64(P + 8 * ((int64_t)qmap[e[p].c] * TILE + e[p].r), val[e[p].k]);
                for (int c = 0; c < TILE; ++c)
                    if (qmap[c] >= 0) P[128 * (int64_t)qn + qmap[c]] = (uint8_t)c;
                break;
            }
            }
            if (ntile == cap_tiles) {
                cap_tiles *= 2;
                int32_t *a1 = realloc(T->tileColIdx, (size_t)cap_tiles * 4);
                if (a1) T->tileColIdx = a1;
                uint8_t *a2 = realloc(T->tileFmt, (size_t)cap_tiles);
                if (a2) T->tileFmt = a2;
                uint8_t *a3 = realloc(T->tileAux, (size_t)cap_tiles);
                if (a3) T->tileAux = a3;
                int32_t *a4 = realloc(held, (size_t)cap_tiles * 4);
                if (a4) held = a4;
                int64_t *a5 = realloc(offs, (size_t)cap_tiles * 8);
                if (a5) offs = a5;
                if (!a1 || !a2 || !a3 || !a4 || !a5) goto fail_free;
            }
            T->tileColIdx[ntile] = ents[a].J;
            T->tileFmt[ntile] = (uint8_t)store_fmt;
            T->tileAux[ntile] = (uint8_t)store_aux;
            held[ntile] = store_nnz;
            offs[ntile] = pay.len / 16;
            T->kept_tiles[store_fmt]++;
            T->kept_nnz[store_fmt] += store_nnz;
            pay.len += sz16;
            ntile++;
            a = b;
        }
    }
    T->tilePtr[T->tilem] = (int32_t)ntile;
    T->numtile = ntile;
    T->tileNnz = malloc((size_t)(ntile + 1) * sizeof(int32_t));
    T->tileOff = malloc((size_t)(ntile + 1) * sizeof(uint32_t));
    if (!T->tileNnz || !T->tileOff) goto fail_free;
    T->tileNnz[0] = 0;
    for (int64_t t = 0; t < ntile; ++t) {
        T->tileNnz[t + 1] = T->tileNnz[t] + held[t];
        T->tileOff[t] = (uint32_t)offs[t];
    }
    T->tileOff[ntile] = (uint32_t)(pay.len / 16);
    T->payload = pay.p ? pay.p : malloc(16);
    T->payload_bytes = pay.len;
    pay.p = NULL;

    /* the extracted entries form a plain CSR matrix in (row, col) order */
    T->remRowPtr = calloc((size_t)(m + 1), sizeof(int32_t));
    int64_t nrem = 0;
    for (int64_t k = 0; k < nnz; ++k) nrem += extracted[k];
    T->remCol = malloc((size_t)(nrem > 0 ? nrem : 1) * sizeof(int32_t));
    T->remVal = malloc((size_t)(nrem > 0 ? nrem : 1) * sizeof(double));
    if (!T->remRowPtr || !T->remCol || !T->remVal) goto fail_free;
    int64_t qr = 0;
    for (int64_t i = 0; i < m; ++i) {
        T->remRowPtr[i] = (int32_t)qr;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k)
            if (extracted[k]) { T->remCol[qr] = colidx[k]; T->remVal[qr] = val[k]; qr++; }
    }
    T->remRowPtr[m] = (int32_t)qr;
    T->rem_nnz = qr;
    free(extracted); free(held); free(offs); free(ents);
    return T;

fail_free:
    free(extracted); free(held); free(offs); free(ents); free(pay.p);
fail:
    oracle_tiling_free(T);
    return NULL;
}

/* ------------------------------------------------------------------------ */
/* Decoder: tiled storage -> (row, col, value) triplets in (row, col) order  */
/* ------------------------------------------------------------------------ */

static double get_f64(const uint8_t *src) { double v; memcpy(&v, src, 8); return v; }
static int get_nibble(const uint8_t *base, int64_t idx)
{ return idx % 2 == 0 ? base[idx / 2] & 15 : base[idx / 2] >> 4; }

typedef struct { int32_t r, c; double v; } trip_t;
static int trip_cmp(const void *a, const void *b)
{
    const trip_t *x = a, *y = b;
    if (x->r != y->r) return x->r < y->r ? -1 : 1;
    if (x->c != y->c) return x->c < y->c ? -1 : 1;
    return 0;
}

/* Writes at most cap triplets; returns the number found (or -1).
 * ELL pads are recognised by R26 (slot k >= 1 with column nibble 0);
 * Dns slots holding +0.0 bits are treated as absent (R27).                 */
int64_t oracle_decode(const oracle_tiling *T, int64_t cap, int32_t *rows,
                      int32_t *cols, double *vals)
{
    int64_t total = T->rem_nnz; /* upper bound on the slots a decode can emit */
    for (int64_t t = 0; t < T->numtile; ++t)
        total += T->tileFmt[t] == O_DNS ? 256
               : T->tileFmt[t] == O_ELL ? 16 * (int64_t)T->tileAux[t]
               : T->tileNnz[t + 1] - T->tileNnz[t];
    trip_t *tr = malloc((size_t)(total > 0 ? total : 1) * sizeof(trip_t));
    if (!tr) return -1;
    int64_t q = 0;
#define EMIT(R, C, V) do { tr[q].r = (R); tr[q].c = (C); tr[q].v = (V); q++; } while (0)
    for (int64_t I = 0; I < T->tilem; ++I)
        for (int64_t t = T->tilePtr[I]; t < T->tilePtr[I + 1]; ++t) {
            const uint8_t *P = T->payload + 16 * (int64_t)T->tileOff[t];
            int64_t nt = T->tileNnz[t + 1] - T->tileNnz[t];
            int32_t R0 = (int32_t)(16 * I), C0 = 16 * T->tileColIdx[t];
            int w = T->tileAux[t];
            switch (T->tileFmt[t]) {
            case O_CSR: {
                const uint8_t *rp = P + 8 * nt;
                for (int r = 0; r < TILE; ++r) {
                    int64_t end = r < 15 ? rp[r + 1] : nt;
                    for (int64_t p = rp[r]; p < end; ++p)
                        EMIT(R0 + r, C0 + get_nibble(P + 8 * nt + 16, p), get_f64(P + 8 * p));
                }
                break;
            }
            case O_COO:
                for (int64_t p = 0; p < nt; ++p)
                    EMIT(R0 + (P[8 * nt + p] >> 4), C0 + (P[8 * nt + p] & 15), get_f64(P + 8 * p));
                break;
            case O_ELL:
                for (int64_t s = 0; s < 16 * (int64_t)w; ++s) {
                    int c = get_nibble(P + 128 * (int64_t)w, s);
                    if (s >= TILE && c == 0) continue; /* pad (R26) */
                    EMIT(R0 + (int32_t)(s % TILE), C0 + c, get_f64(P + 8 * s));
                }
                break;
            case O_HYB: {
                int64_t kc = nt - 16 * (int64_t)w;
                const uint8_t *coov = P + 128 * (int64_t)w, *elli = coov + 8 * kc,
                              *cooi = elli + 8 * (int64_t)w;
                for (int64_t s = 0; s < 16 * (int64_t)w; ++s)
                    EMIT(R0 + (int32_t)(s % TILE), C0 + get_nibble(elli, s), get_f64(P + 8 * s));
                for (int64_t p = 0; p < kc; ++p)
                    EMIT(R0 + (cooi[p] >> 4), C0 + (cooi[p] & 15), get_f64(coov + 8 * p));
                break;
            }
            case O_DNS:
                for (int64_t s = 0; s < 256; ++s) {
                    uint64_t bits;
                    memcpy(&bits, P + 8 * s, 8);
                    if (bits == 0) continue; /* +0.0 fill (R27) */
                    EMIT(R0 + (int32_t)(s % TILE), C0 + (int32_t)(s / TILE), get_f64(P + 8 * s));
                }
                break;
            case O_DNSROW:
                for (int qq = 0; qq < w; ++qq)
                    for (int c = 0; c < TILE; ++c)
                        EMIT(R0 + P[128 * w + qq], C0 + c, get_f64(P + 8 * (qq * TILE + c)));
                break;
            case O_DNSCOL:
                for (int qq = 0; qq < w; ++qq)
                    for (int r = 0; r < TILE; ++r)
                        EMIT(R0 + r, C0 + P[128 * w + qq], get_f64(P + 8 * (qq * TILE + r)));
                break;
            }
        }
    for (int64_t i = 0; i < T->m; ++i)
        for (int64_t k = T->remRowPtr[i]; k < T->remRowPtr[i + 1]; ++k)
            EMIT((int32_t)i, T->remCol[k], T->remVal[k]);
#undef EMIT
    qsort(tr, (size_t)q, sizeof(trip_t), trip_cmp);
    for (int64_t p = 0; p < q && p < cap; ++p) { rows[p] = tr[p].r; cols[p] = tr[p].c; vals[p] = tr[p].v; }
    free(tr);
    return q;
}

/* ------------------------------------------------------------------------ */
/* accessors for the ctypes wrapper (oracle/oracle.py)                       */
/* ------------------------------------------------------------------------ */

int64_t oracle_tiling_scalar(const oracle_tiling *T, int32_t which)
{
    switch (which) {
    case 0: return T->m;
    case 1: return T->n;
    case 2: return T->nnz;
    case 3: return T->tilem;
    case 4: return T->tilen;
    case 5: return T->mode;
    case 6: return T->numtile;
    case 7: return T->payload_bytes;
    case 8: return T->rem_nnz;
    default:
        if (which >= 100 && which < 107) return T->sel_tiles[which - 100];
        if (which >= 110 && which < 117) return T->sel_nnz[which - 110];
        if (which >= 120 && which < 127) return T->kept_tiles[which - 120];
        if (which >= 130 && which < 137) return T->kept_nnz[which - 130];
        return -1;
    }
}

const void *oracle_tiling_array(const oracle_tiling *T, int32_t which)
{
    switch (which) {
    case 0: return T->tilePtr;
    case 1: return T->tileColIdx;
    case 2: return T->tileNnz;
    case 3: return T->tileFmt;
    case 4: return T->tileAux;
    case 5: return T->tileOff;
    case 6: return T->payload;
    case 7: return T->remRowPtr;
    case 8: return T->remCol;
    case 9: return T->remVal;
    default: return NULL;
    }
}
