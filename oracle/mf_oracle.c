/*
 * mf_oracle.c -- the ORACLE for the Mille-feuille hot path (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares no code, header, table or constant generator
 * with the CUDA path under paper_conf_sc_yangznjs0t024_b200/csrc; neither side
 * includes the other.
 *
 * What it is: a plain, slow, obviously-correct CPU implementation in IEEE binary64
 * of what the method computes, written from PAPER.md ("P:<line>" cites
 * /root/reference/PAPER.md).  Readings of garbled / silent passages follow
 * SURVEY.md section 8(c) and are listed in DESIGN.md ("Readings").
 *
 * Build: gcc -O2 -std=c11 -fPIC -shared -ffp-contract=off -o liboracle.so mf_oracle.c -lm
 * -ffp-contract=off matters: every fused multiply-add below is an explicit fma();
 * no other expression may be contracted.
 *
 * Pins (tests/test_oracle_*.py) -- what fixes each function other than itself:
 *   orc_rne / orc_classify      closed-form test vectors (SURVEY c-2), brute force over all
 *                               E4M3 / FP16 bit patterns, numpy float32/float16 casts.
 *   orc_tiles_build             dense round trip, brute force over every 2x2 / 3x3 pattern
 *                               (T=2,3), Fig. 6 structure.
 *   orc_levels / orc_tile_eff   Fig. 7 replay: 6, 8, 9 lowered, 6 bypassed.
 *   orc_spmv_tiles              numpy dense A~ v built independently, exact.
 *   orc_dot                     math.fsum within n*eps; plain == textbook fma chain.
 *   orc_cg / orc_bicgstab       numpy.linalg.solve, finite termination, A-orthogonality,
 *                               recurrence gap, x* = 1.
 *   orc_ilu0 / orc_ilu_apply    tridiagonal ILU(0) == exact LU; (LU)_ij == A_ij on pattern.
 *   rb_lower / rb_upper         (recursive block SpTRSV) exact integer triangular systems
 *                               solved in Python integers; scipy-free dense back substitution
 *                               within the forward-error bound; depth 0 == substitution.
 *   orc_pcg / orc_pbicgstab     numpy.linalg.solve on small systems.
 * The dynamic switch's effect on iteration counts is "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* status codes: same numbering as the boundary's mf_status (declared independently) */
enum { ORC_OK = 0, ORC_ERR_INVALID_ARG = 1, ORC_ERR_UNSORTED_CSR = 2, ORC_ERR_NONFINITE = 3,
       ORC_ERR_OOM = 4, ORC_ERR_BREAKDOWN = 7, ORC_ERR_ZERO_PIVOT = 8 };

/* precision codes: larger = lower precision (SURVEY 8b mf_prec); 4 = bypass (D6) */
enum { P_FP64 = 0, P_FP32 = 1, P_FP16 = 2, P_FP8 = 3, P_BYPASS = 4 };

/* ------------------------------------------------------------------------------------
 * 1. Rounding to the lower formats ("store each nonzero in four data types").
 *    Reading c-8 #4: a SINGLE round-to-nearest-even from the binary64 value.
 *    Formats: FP32 = IEEE binary32; FP16 = IEEE binary16; FP8 = OCP E4M3FN (c-8 #2),
 *    which has no infinity -- overflow saturates to +-448 (satfinite).
 *    Implementation by exact power-of-two scaling: |v| = s * 2^q with q the quantum
 *    exponent of the target format at |v|'s binade; s is rounded to an integer (RNE).
 * ---------------------------------------------------------------------------------- */
typedef struct { int p; int emin; double maxf; int saturate; } orc_fmt;

static orc_fmt fmt_of(int prec) {
    orc_fmt f;
    switch (prec) {
    case P_FP32: f.p = 24; f.emin = -126; f.maxf = ldexp(2.0 - ldexp(1.0, -23), 127); f.saturate = 0; break;
    case P_FP16: f.p = 11; f.emin = -14;  f.maxf = 65504.0; f.saturate = 0; break;
    default:     f.p = 4;  f.emin = -6;   f.maxf = 448.0;   f.saturate = 1; break; /* E4M3FN */
    }
    return f;
}

double orc_rne(double v, int prec) {
    if (prec == P_FP64 || v == 0.0 || isnan(v)) return v;
    orc_fmt f = fmt_of(prec);
    if (isinf(v)) return f.saturate ? copysign(f.maxf, v) : v;
    double a = fabs(v);
    int e = ilogb(a);                 /* a in [2^e, 2^(e+1)) */
    if (e < f.emin) e = f.emin;       /* subnormal range: fixed quantum */
    int q = e - (f.p - 1);            /* quantum exponent */
    double s = ldexp(a, -q);          /* exact: power-of-two scaling, s < 2^p */
    double fl = floor(s);
    double frac = s - fl;             /* exact */
    if (frac > 0.5 || (frac == 0.5 && fmod(fl, 2.0) == 1.0)) fl += 1.0;
    double r = ldexp(fl, q);
    if (r > f.maxf) r = f.saturate ? f.maxf : INFINITY;
    return copysign(r, v);
}

/* bit encodings of values already representable in the format */
uint16_t orc_fp16_bits(double r) {
    uint16_t s = signbit(r) ? 0x8000u : 0u;
    double a = fabs(r);
    if (isnan(r)) return 0x7E00u;
    if (isinf(a)) return (uint16_t)(s | 0x7C00u);
    if (a == 0.0) return s;
    if (a < ldexp(1.0, -14)) return (uint16_t)(s | (uint16_t)ldexp(a, 24));      /* subnormal */
    int e = ilogb(a);
    uint16_t mant = (uint16_t)(ldexp(a, -e) * 1024.0 - 1024.0);
    return (uint16_t)(s | (uint16_t)((e + 15) << 10) | mant);
}
double orc_fp16_value(uint16_t b) {
    int s = b >> 15, ex = (b >> 10) & 31, m = b & 1023;
    double v;
    if (ex == 31) v = m ? NAN : INFINITY;
    else if (ex == 0) v = ldexp((double)m, -24);
    else v = ldexp(1.0 + m / 1024.0, ex - 15);
    return s ? -v : v;
}
uint8_t orc_e4m3_bits(double r) {
    uint8_t s = signbit(r) ? 0x80u : 0u;
    double a = fabs(r);
    if (isnan(r)) return 0x7Fu;
    if (a == 0.0) return s;
    if (a < ldexp(1.0, -6)) return (uint8_t)(s | (uint8_t)ldexp(a, 9));          /* subnormal */
    int e = ilogb(a);
    uint8_t mant = (uint8_t)(ldexp(a, -e) * 8.0 - 8.0);
    return (uint8_t)(s | (uint8_t)((e + 7) << 3) | mant);
}
double orc_e4m3_value(uint8_t b) {
    int s = b >> 7, ex = (b >> 3) & 15, m = b & 7;
    double v;
    if (ex == 15 && m == 7) v = NAN;
    else if (ex == 0) v = ldexp((double)m, -9);
    else v = ldexp(1.0 + m / 8.0, ex - 7);
    return s ? -v : v;
}

/* ------------------------------------------------------------------------------------
 * 2. Per-nonzero precision criterion (Section II-A).
 *    "compute the loss between three lower precisions ... and the FP64. If the losses
 *    ... are less than 10^-15 ... the nonzero will be stored in the lowest possible
 *    precision."  Reading c-8 #1: relative loss, |v - RNE_q(v)| < 1e-15 |v|; v = 0 -> FP8.
 * ---------------------------------------------------------------------------------- */
int orc_classify(double v, double loss_tol) {
    if (v == 0.0) return P_FP8;
    for (int q = P_FP8; q >= P_FP32; --q) {
        double r = orc_rne(v, q);
        double loss = fabs(v - r);
        if (loss < loss_tol * fabs(v)) return q;
    }
    return P_FP64;
}

/* normal range [min_normal_q, max_q] of format q (for the range floor, c-1.7) */
static int in_normal_range(double a, int q) {
    switch (q) {
    case P_FP32: return a >= ldexp(1.0, -126) && a <= ldexp(2.0 - ldexp(1.0, -23), 127);
    case P_FP16: return a >= ldexp(1.0, -14) && a <= 65504.0;
    case P_FP8:  return a >= ldexp(1.0, -6) && a <= 448.0;
    default:     return 1;
    }
}

/* ------------------------------------------------------------------------------------
 * 3. Two-level tile format (Section III-B, Fig. 5; canonical form SURVEY c-1).
 *    High level (COO of tiles): TileRowidx, TileColidx, TilePrec [tilenum];
 *    TileNnz, Nonrow [tilenum+1] (offsets of nonzeros / non-empty rows).
 *    Low level (CSR inside each tile): RowIndex, CsrRowptr [rownum]; CsrColidx [nnz];
 *    values in four typed arrays Val64/Val32/Val16/Val8, tile t's values contiguous in
 *    the array of its precision starting at ValOff[t].  TileRowPtr = CSR-of-tiles view.
 * ---------------------------------------------------------------------------------- */
typedef struct {
    int64_t n_rows, n_cols, nnz;
    int32_t T;
    int64_t tilenum, rownum, n_tile_rows;
    int32_t *TileRowidx, *TileColidx;
    uint8_t *TilePrec, *Floor;
    int64_t *TileNnz, *Nonrow, *ValOff, *TileRowPtr;
    uint8_t *RowIndex, *CsrRowptr, *CsrColidx;
    double *Val64;
    float *Val32;
    uint16_t *Val16;
    uint8_t *Val8;
    int64_t nval[4];
} orc_tiles;

void orc_tiles_free(orc_tiles* A) {
    if (!A) return;
    free(A->TileRowidx); free(A->TileColidx); free(A->TilePrec); free(A->Floor);
    free(A->TileNnz); free(A->Nonrow); free(A->ValOff); free(A->TileRowPtr);
    free(A->RowIndex); free(A->CsrRowptr); free(A->CsrColidx);
    free(A->Val64); free(A->Val32); free(A->Val16); free(A->Val8);
    memset(A, 0, sizeof(*A));
}

static int cmp_i64(const void* a, const void* b) {
    int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
    return (x > y) - (x < y);
}

/* validate CSR: rowptr monotone from 0 to nnz, columns strictly increasing in [0,n_cols), finite */
int orc_csr_validate(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* rowptr,
                     const int32_t* colidx, const double* vals) {
    if (n_rows < 0 || n_cols < 0 || nnz < 0 || !rowptr) return ORC_ERR_INVALID_ARG;
    if (rowptr[0] != 0 || rowptr[n_rows] != nnz) return ORC_ERR_INVALID_ARG;
    for (int64_t i = 0; i < n_rows; ++i) {
        if (rowptr[i + 1] < rowptr[i]) return ORC_ERR_INVALID_ARG;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) {
            if (colidx[k] < 0 || colidx[k] >= n_cols) return ORC_ERR_INVALID_ARG;
            if (k > rowptr[i] && colidx[k] <= colidx[k - 1]) return ORC_ERR_UNSORTED_CSR;
        }
    }
    for (int64_t k = 0; k < nnz; ++k)
        if (!isfinite(vals[k])) return ORC_ERR_NONFINITE;
    return ORC_OK;
}

/* growable array helper: ensures capacity for `need` elements of `esz` bytes */
static int grow(void** p, int64_t* cap, int64_t need, size_t esz) {
    if (need <= *cap) return 1;
    int64_t nc = *cap ? *cap : 1024;
    while (nc < need) nc *= 2;
    void* np = realloc(*p, (size_t)nc * esz);
    if (!np) return 0;
    *p = np; *cap = nc;
    return 1;
}
#define GROW(ptr, cap, need) do { if (!grow((void**)&(ptr), &(cap), (need), sizeof(*(ptr)))) { st = ORC_ERR_OOM; goto fail; } } while (0)

int orc_tiles_build(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* rowptr,
                    const int32_t* colidx, const double* vals, int32_t T, int classify,
                    double loss_tol, orc_tiles* A) {
    memset(A, 0, sizeof(*A));
    if (T < 1 || T > 16) return ORC_ERR_INVALID_ARG;
    int st = orc_csr_validate(n_rows, n_cols, nnz, rowptr, colidx, vals);
    if (st != ORC_OK) return st;
    A->n_rows = n_rows; A->n_cols = n_cols; A->nnz = nnz; A->T = T;
    A->n_tile_rows = (n_rows + T - 1) / T;
    /* capacities: per-tile arrays, offsets arrays, per-row arrays, value arrays */
    int64_t c_trow = 0, c_tcol = 0, c_prec = 0, c_floor = 0, c_voff = 0, c_tnnz = 0, c_nonrow = 0;
    int64_t c_ridx = 0, c_rptr = 0, c_v[4] = {0, 0, 0, 0}, c_tc = 0;
    int64_t* tcols = NULL;
    int64_t* cursor = (int64_t*)malloc(sizeof(int64_t) * (size_t)T);
    double* tv = (double*)malloc(sizeof(double) * (size_t)T * (size_t)T);   /* one tile's values */
    A->TileRowPtr = (int64_t*)calloc((size_t)A->n_tile_rows + 1, sizeof(int64_t));
    A->CsrColidx = (uint8_t*)malloc((size_t)(nnz > 0 ? nnz : 1));
    if (!cursor || !tv || !A->TileRowPtr || !A->CsrColidx) { st = ORC_ERR_OOM; goto fail; }
    GROW(A->TileNnz, c_tnnz, 1);
    GROW(A->Nonrow, c_nonrow, 1);
    A->TileNnz[0] = 0; A->Nonrow[0] = 0;
    int64_t t = 0, ri = 0, k_out = 0;
    for (int64_t TR = 0; TR < A->n_tile_rows; ++TR) {
        int64_t r0 = TR * T, r1 = r0 + T < n_rows ? r0 + T : n_rows;
        /* the distinct tile columns of this tile row, ascending */
        int64_t cnt = 0;
        for (int64_t i = r0; i < r1; ++i) {
            GROW(tcols, c_tc, cnt + (rowptr[i + 1] - rowptr[i]) + 1);
            for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) tcols[cnt++] = colidx[k] / T;
        }
        if (cnt) qsort(tcols, (size_t)cnt, sizeof(int64_t), cmp_i64);
        int64_t nd = 0;
        for (int64_t a = 0; a < cnt; ++a) if (nd == 0 || tcols[a] != tcols[nd - 1]) tcols[nd++] = tcols[a];
        for (int64_t i = r0; i < r1; ++i) cursor[i - r0] = rowptr[i];
        for (int64_t d = 0; d < nd; ++d, ++t) {
            int64_t tc = tcols[d];
            GROW(A->TileRowidx, c_trow, t + 1);
            GROW(A->TileColidx, c_tcol, t + 1);
            GROW(A->TilePrec, c_prec, t + 1);
            GROW(A->Floor, c_floor, t + 1);
            GROW(A->ValOff, c_voff, t + 1);
            GROW(A->TileNnz, c_tnnz, t + 2);
            GROW(A->Nonrow, c_nonrow, t + 2);
            A->TileRowidx[t] = (int32_t)TR;
            A->TileColidx[t] = (int32_t)tc;
            int64_t nz = 0;
            int best = classify ? P_FP8 : P_FP64;
            for (int64_t i = r0; i < r1; ++i) {           /* local rows ascending */
                int64_t k = cursor[i - r0];
                if (k >= rowptr[i + 1] || colidx[k] / T != tc) continue;   /* row empty in tile */
                GROW(A->RowIndex, c_ridx, ri + 1);
                GROW(A->CsrRowptr, c_rptr, ri + 1);
                A->RowIndex[ri] = (uint8_t)(i - r0);
                A->CsrRowptr[ri] = (uint8_t)nz;
                ++ri;
                for (; k < rowptr[i + 1] && colidx[k] / T == tc; ++k) {   /* columns ascending */
                    A->CsrColidx[k_out++] = (uint8_t)(colidx[k] % T);
                    tv[nz++] = vals[k];
                    if (classify) { int c = orc_classify(vals[k], loss_tol); if (c < best) best = c; }
                }
                cursor[i - r0] = k;
            }
            A->TileNnz[t + 1] = A->TileNnz[t] + nz;
            A->Nonrow[t + 1] = ri;
            /* TilePrec: the highest precision any nonzero of the tile needs (c-8 #3) */
            A->TilePrec[t] = (uint8_t)best;
            /* stored values RNE_TilePrec(v), appended to the array of that precision (c-1.6) */
            int64_t off = A->nval[best];
            A->ValOff[t] = off;
            switch (best) {
            case P_FP64: GROW(A->Val64, c_v[0], off + nz);
                { for (int64_t a = 0; a < nz; ++a) A->Val64[off + a] = tv[a]; }
                break;
            case P_FP32: GROW(A->Val32, c_v[1], off + nz);
                { for (int64_t a = 0; a < nz; ++a) A->Val32[off + a] = (float)orc_rne(tv[a], P_FP32); }
                break;
            case P_FP16: GROW(A->Val16, c_v[2], off + nz);
                { for (int64_t a = 0; a < nz; ++a) A->Val16[off + a] = orc_fp16_bits(orc_rne(tv[a], P_FP16)); }
                break;
            default:     GROW(A->Val8, c_v[3], off + nz);
                { for (int64_t a = 0; a < nz; ++a) A->Val8[off + a] = orc_e4m3_bits(orc_rne(tv[a], P_FP8)); }
                break;
            }
            A->nval[best] += nz;
            /* range floor (c-1.7): the lowest q at or below TilePrec whose normal range holds
             * every nonzero stored |v| (zeros round exactly in every format: ignored) */
            int fl = best;
            for (int q = P_FP8; q > best; --q) {
                int ok = 1;
                for (int64_t a = 0; a < nz && ok; ++a) {
                    double sv = orc_rne(tv[a], best);
                    if (sv != 0.0 && !in_normal_range(fabs(sv), q)) ok = 0;
                }
                if (ok) { fl = q; break; }
            }
            A->Floor[t] = (uint8_t)fl;
        }
        A->TileRowPtr[TR + 1] = t;
    }
    A->tilenum = t; A->rownum = ri;
    free(cursor); free(tcols); free(tv);
    return ORC_OK;
fail:
    free(cursor); free(tcols); free(tv);
    orc_tiles_free(A);
    return st;
}

/* stored value of the a-th nonzero of tile t, decoded exactly to binary64 */
double orc_tile_value(const orc_tiles* A, int64_t t, int64_t a) {
    int64_t o = A->ValOff[t] + a;
    switch (A->TilePrec[t]) {
    case P_FP64: return A->Val64[o];
    case P_FP32: return (double)A->Val32[o];
    case P_FP16: return orc_fp16_value(A->Val16[o]);
    default:     return orc_e4m3_value(A->Val8[o]);
    }
}

/* stored values back to a row-major CSR (same pattern as the input CSR) */
void orc_tiles_stored_csr(const orc_tiles* A, const int64_t* rowptr, int32_t* colidx_out, double* vals_out) {
    int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)(A->n_rows > 0 ? A->n_rows : 1));
    for (int64_t i = 0; i < A->n_rows; ++i) fill[i] = rowptr[i];
    for (int64_t t = 0; t < A->tilenum; ++t) {
        for (int64_t ri = A->Nonrow[t]; ri < A->Nonrow[t + 1]; ++ri) {
            int64_t row = (int64_t)A->TileRowidx[t] * A->T + A->RowIndex[ri];
            int64_t s = A->CsrRowptr[ri];
            int64_t e = (ri + 1 < A->Nonrow[t + 1]) ? A->CsrRowptr[ri + 1] : A->TileNnz[t + 1] - A->TileNnz[t];
            for (int64_t a = s; a < e; ++a) {
                colidx_out[fill[row]] = (int32_t)((int64_t)A->TileColidx[t] * A->T + A->CsrColidx[A->TileNnz[t] + a]);
                vals_out[fill[row]] = orc_tile_value(A, t, a);
                fill[row]++;
            }
        }
    }
    free(fill);
}

/* ------------------------------------------------------------------------------------
 * 4. Convergent-element retrieval (Alg. 4) and the effective tile precision
 *    (Alg. 5 l.2-4).  Thresholds th = {tau*1e-3, tau*1e-2, tau*1e-1, tau} (Alg. 4 l.1).
 *    |p| < th0 -> bypass; [th0,th1) -> FP8; [th1,th2) -> FP16; [th2,th3) -> FP32.
 *    Readings: c-8 #5 (follow P:174, not Alg. 4's u+1), #7 (|p|), #18 (tail segment).
 * ---------------------------------------------------------------------------------- */
void orc_levels(const double* v, int64_t n, int32_t T, const double th[4], uint8_t* level) {
    int64_t nseg = (n + T - 1) / T;
    for (int64_t J = 0; J < nseg; ++J) {
        double m = 0.0;
        int nan = 0;
        for (int64_t k = J * T; k < (J + 1) * T && k < n; ++k) {
            if (isnan(v[k])) nan = 1;
            else if (fabs(v[k]) > m) m = fabs(v[k]);
        }
        uint8_t lv;
        if (nan) lv = P_FP64;
        else if (m < th[0]) lv = P_BYPASS;
        else if (m < th[1]) lv = P_FP8;
        else if (m < th[2]) lv = P_FP16;
        else if (m < th[3]) lv = P_FP32;
        else lv = P_FP64;
        level[J] = lv;
    }
}

/* e_t (SURVEY c-5): bypass if the column segment is bypassed; otherwise the lower of
 * (TilePrec, level) -- but never below the tile's range floor when range_guard is set. */
static int tile_eff(const orc_tiles* A, int64_t t, const uint8_t* level, int range_guard, const uint8_t* cur) {
    int lv = level ? level[A->TileColidx[t]] : P_FP64;
    if (lv == P_BYPASS) return P_BYPASS;
    int base = cur ? cur[t] : A->TilePrec[t];
    int e = lv > base ? lv : base;                     /* min_prec = larger code */
    if (range_guard && e > A->Floor[t]) e = A->Floor[t]; /* max_prec with the floor */
    return e;
}

void orc_tile_eff(const orc_tiles* A, const uint8_t* level, int range_guard, uint8_t* out) {
    for (int64_t t = 0; t < A->tilenum; ++t) out[t] = (uint8_t)tile_eff(A, t, level, range_guard, NULL);
}

/* ------------------------------------------------------------------------------------
 * 5. Mixed-precision tiled SpMV (Alg. 5).  For each tile: bypass or compute
 *    with its values at e_t (val_eff = RNE_{e_t}(stored), upcast exactly, c-8 #10).
 *    Every row is ONE fma chain in ascending column order starting from +0 (SURVEY c-3);
 *    tiles of a tile row are visited in ascending tile column, so a row's entries are
 *    visited in ascending column.  Bypassed tiles contribute nothing (skipped, not 0*x).
 *    Sticky state (P:237 literal; c-5 "sticky variant"): cur[t] and the working copy wv[]
 *    (values in tile order, per nonzero) are lowered in place by successive rounding.
 * ---------------------------------------------------------------------------------- */
typedef struct { uint8_t* cur; double* wv; } orc_sticky;

/* decoded stored values in tile order (a cache of orc_tile_value; no arithmetic) */
double* orc_decode_values(const orc_tiles* A) {
    double* sv = (double*)malloc(sizeof(double) * (size_t)(A->nnz > 0 ? A->nnz : 1));
    if (!sv) return NULL;
    for (int64_t t = 0; t < A->tilenum; ++t)
        for (int64_t a = 0; a < A->TileNnz[t + 1] - A->TileNnz[t]; ++a) sv[A->TileNnz[t] + a] = orc_tile_value(A, t, a);
    return sv;
}

static void spmv_tiles(const orc_tiles* A, const double* sv, const double* x, double* y, const uint8_t* level,
                       int range_guard, orc_sticky* sticky, int64_t counts[5]) {
    int32_t T = A->T;
    double acc[16];
    for (int64_t TR = 0; TR < A->n_tile_rows; ++TR) {
        for (int r = 0; r < T; ++r) acc[r] = 0.0;
        for (int64_t t = A->TileRowPtr[TR]; t < A->TileRowPtr[TR + 1]; ++t) {
            int e = tile_eff(A, t, level, range_guard, sticky ? sticky->cur : NULL);
            if (counts) counts[e]++;
            if (e == P_BYPASS) continue;
            if (sticky && e > sticky->cur[t]) {            /* one-time in-place downgrade */
                for (int64_t a = A->TileNnz[t]; a < A->TileNnz[t + 1]; ++a) sticky->wv[a] = orc_rne(sticky->wv[a], e);
                sticky->cur[t] = (uint8_t)e;
            }
            for (int64_t ri = A->Nonrow[t]; ri < A->Nonrow[t + 1]; ++ri) {
                int lr = A->RowIndex[ri];
                int64_t s = A->CsrRowptr[ri];
                int64_t en = (ri + 1 < A->Nonrow[t + 1]) ? A->CsrRowptr[ri + 1] : A->TileNnz[t + 1] - A->TileNnz[t];
                for (int64_t a = s; a < en; ++a) {
                    int64_t col = (int64_t)A->TileColidx[t] * T + A->CsrColidx[A->TileNnz[t] + a];
                    double v;
                    if (sticky) v = sticky->wv[A->TileNnz[t] + a];
                    else {
                        double s0 = sv ? sv[A->TileNnz[t] + a] : orc_tile_value(A, t, a);
                        v = (e == A->TilePrec[t]) ? s0 : orc_rne(s0, e);   /* RNE_TilePrec(s0) == s0 */
                    }
                    acc[lr] = fma(v, x[col], acc[lr]);
                }
            }
        }
        for (int r = 0; r < T && TR * T + r < A->n_rows; ++r) y[TR * T + r] = acc[r];
    }
}

void orc_spmv_tiles(const orc_tiles* A, const double* x, double* y, const uint8_t* level,
                    int range_guard, orc_sticky* sticky, int64_t counts[5]) {
    spmv_tiles(A, NULL, x, y, level, range_guard, sticky, counts);
}

/* plain CSR SpMV: one fma chain per row, ascending column */
void orc_spmv_csr(int64_t n, const int64_t* rowptr, const int32_t* colidx, const double* vals,
                  const double* x, double* y) {
    for (int64_t i = 0; i < n; ++i) {
        double acc = 0.0;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) acc = fma(vals[k], x[colidx[k]], acc);
        y[i] = acc;
    }
}

/* ------------------------------------------------------------------------------------
 * 6. Dot products (Alg. 1 l.5, l.9; Alg. 3 steps B/C block-level reduction).
 *    plan == NULL: plain sequential fma chain.
 *    plan != NULL: the kernel-order tree of SURVEY c-7 (a reading: the paper fixes no
 *    summation order).  G CTAs, CTA g owns rows [R[g], R[g+1]); B threads per CTA:
 *      thread t: acc = fma(u_i, v_i, acc) over i = R[g]+t, R[g]+t+B, ...  (from +0)
 *      warp:     xor-butterfly over offsets 16,8,4,2,1 (lane l: v[l] + v[l^o])
 *      CTA:      tree32 over the W = B/32 warp totals
 *      grid:     tree32 over the G CTA totals
 *    tree32(x[0..c)): lane l sums x[l], x[l+32], ... left to right from +0, then butterfly.
 *    Row-block ranks (P > 0, the rows of rank q are those of CTAs [Gr[q], Gr[q+1])):
 *      rank q:   tree32 over its CTA totals (the grid level of q's own launch)
 *      total:    ((+0 + rank_0) + rank_1) + ... in rank order
 *    (again a reading: the paper is single-GPU.)
 * ---------------------------------------------------------------------------------- */
typedef struct { int32_t G; int32_t B; const int64_t* R; int32_t P; const int32_t* Gr; } orc_plan;

static double butterfly32(double* v) {
    double nv[32];
    for (int o = 16; o >= 1; o >>= 1) {
        for (int l = 0; l < 32; ++l) nv[l] = v[l] + v[l ^ o];
        memcpy(v, nv, sizeof(nv));
    }
    return v[0];
}

static double tree32(const double* x, int64_t c) {
    double s[32];
    for (int l = 0; l < 32; ++l) {
        s[l] = 0.0;
        for (int64_t m = l; m < c; m += 32) s[l] = s[l] + x[m];
    }
    return butterfly32(s);
}

double orc_dot(const double* u, const double* v, int64_t n, const orc_plan* plan) {
    if (!plan) {
        double acc = 0.0;
        for (int64_t i = 0; i < n; ++i) acc = fma(u[i], v[i], acc);
        return acc;
    }
    int32_t W = plan->B / 32;
    double* slot = (double*)malloc(sizeof(double) * (size_t)plan->G);
    double* wt = (double*)malloc(sizeof(double) * (size_t)W);
    for (int32_t g = 0; g < plan->G; ++g) {
        int64_t end = plan->R[g + 1] < n ? plan->R[g + 1] : n;
        for (int32_t w = 0; w < W; ++w) {
            double lane[32];
            for (int l = 0; l < 32; ++l) {
                double acc = 0.0;
                for (int64_t i = plan->R[g] + 32 * w + l; i < end; i += plan->B) acc = fma(u[i], v[i], acc);
                lane[l] = acc;
            }
            wt[w] = butterfly32(lane);
        }
        slot[g] = tree32(wt, W);
    }
    double r;
    if (plan->P > 0) {
        r = 0.0;
        for (int32_t q = 0; q < plan->P; ++q) r = r + tree32(slot + plan->Gr[q], plan->Gr[q + 1] - plan->Gr[q]);
    } else {
        r = tree32(slot, plan->G);
    }
    free(slot); free(wt);
    return r;
}

/* ------------------------------------------------------------------------------------
 * 7. Solvers.  CG = Alg. 1 in canonical order (SURVEY c-3); BiCGSTAB = Alg. 2
 *    with the sign of s corrected (c-8 #12).  Stop on ||r||/||b|| < tol (c-8 #8),
 *    max_iter.  Switch thresholds tau = switch_eps * ||v0||_2 (v0 = first SpMV input;
 *    reading R8) or tau = switch_eps when switch_absolute (Alg. 1 l.3 literal).
 * ---------------------------------------------------------------------------------- */
enum { MODE_FP64 = 0, MODE_STATIC = 1, MODE_DYNAMIC = 2 };

typedef struct {
    double tol; int64_t max_iter; int32_t mode; double switch_eps;
    int32_t switch_absolute; int32_t sticky; int32_t range_guard;
} orc_opts;

typedef struct {
    int64_t iterations; int32_t converged; int32_t status; double rel_residual;
    int64_t n_spmv;
} orc_info;

typedef struct {            /* optional ILU(0) preconditioner (CSR, L\U in one array) */
    int64_t n; const int64_t* rowptr; const int32_t* colidx; const double* lu; const int64_t* diag;
    int32_t rb_depth;       /* 0: row-by-row substitution; d > 0: recursive block SpTRSV of depth d */
} orc_ilu;

static void ilu_apply(const orc_ilu* M, const double* r, double* z);

typedef struct {
    const orc_tiles* A; const orc_opts* o; const orc_plan* plan;
    orc_sticky sticky; int use_sticky;
    double th[4]; uint8_t* level; double* sv;
    int64_t* level_counts; int64_t lc_cap; int64_t n_spmv;
} orc_ctx;

/* tau (reading R8 in DESIGN.md; SURVEY c-5): P:174 compares the entries of p_j with "the
 * convergence threshold eps"; the stop test is relative, ||r|| < eps ||b||, so in the
 * units of the SpMV input the threshold is eps times the norm of the first SpMV input v0
 * (= ||b|| for CG with x0 = 0):  tau = switch_eps * ||v0||_2;  switch_absolute: tau = switch_eps
 * (Alg. 1 l.3 literal).  Default switch_eps = tol. */
static void ctx_set_tau(orc_ctx* c, double vnorm) {
    double tau = c->o->switch_absolute ? c->o->switch_eps : c->o->switch_eps * vnorm;
    c->th[0] = tau * 1e-3; c->th[1] = tau * 1e-2; c->th[2] = tau * 1e-1; c->th[3] = tau;
}

static void ctx_spmv(orc_ctx* c, const double* v, double* out) {
    const uint8_t* lv = NULL;
    if (c->o->mode == MODE_DYNAMIC) { orc_levels(v, c->A->n_cols, c->A->T, c->th, c->level); lv = c->level; }
    int64_t cnt[5] = {0, 0, 0, 0, 0};
    spmv_tiles(c->A, c->sv, v, out, lv, c->o->range_guard, c->use_sticky ? &c->sticky : NULL, cnt);
    if (c->level_counts && c->n_spmv < c->lc_cap)
        for (int q = 0; q < 5; ++q) c->level_counts[5 * c->n_spmv + q] = cnt[q];
    c->n_spmv++;
}

static int ctx_init(orc_ctx* c, const orc_tiles* A, const orc_opts* o, const orc_plan* plan,
                    int64_t* level_counts, int64_t lc_cap) {
    memset(c, 0, sizeof(*c));
    c->A = A; c->o = o; c->plan = plan; c->level_counts = level_counts; c->lc_cap = lc_cap;
    c->level = (uint8_t*)calloc((size_t)((A->n_cols + A->T - 1) / A->T + 1), 1);
    c->sv = orc_decode_values(A);
    if (o->mode == MODE_DYNAMIC && o->sticky) {
        c->use_sticky = 1;
        c->sticky.cur = (uint8_t*)malloc((size_t)(A->tilenum + 1));
        c->sticky.wv = (double*)malloc(sizeof(double) * (size_t)(A->nnz + 1));
        for (int64_t t = 0; t < A->tilenum; ++t) {
            c->sticky.cur[t] = A->TilePrec[t];
            for (int64_t a = 0; a < A->TileNnz[t + 1] - A->TileNnz[t]; ++a)
                c->sticky.wv[A->TileNnz[t] + a] = orc_tile_value(A, t, a);
        }
    }
    return (c->level && c->sv) ? ORC_OK : ORC_ERR_OOM;
}

static void ctx_free(orc_ctx* c) { free(c->level); free(c->sv); free(c->sticky.cur); free(c->sticky.wv); }

static int all_zero(const double* x, int64_t n) {
    for (int64_t i = 0; i < n; ++i) if (x[i] != 0.0) return 0;
    return 1;
}

/* r = b - A x0 with the stored values at TilePrec (x0 == 0 -> r = b exactly) */
static void initial_residual(const orc_tiles* A, const double* b, const double* x, double* r) {
    int64_t n = A->n_rows;
    if (all_zero(x, n)) { memcpy(r, b, sizeof(double) * (size_t)n); return; }
    orc_spmv_tiles(A, x, r, NULL, 0, NULL, NULL);
    for (int64_t i = 0; i < n; ++i) r[i] = b[i] - r[i];
}

static void record(double* hist, int64_t cap, int64_t j, double v) { if (hist && j < cap) hist[j] = v; }

/* CG (and PCG when M != NULL: z = M^-1 r, rho = (r,z), p = z + beta p; SURVEY c-6) */
int orc_pcg(const orc_tiles* A, const orc_ilu* M, const double* b, double* x, const orc_opts* o,
            const orc_plan* plan, double* hist, int64_t hist_cap, int64_t* level_counts,
            int64_t lc_cap, orc_info* info) {
    int64_t n = A->n_rows;
    if (A->n_rows != A->n_cols) return ORC_ERR_INVALID_ARG;
    orc_ctx c;
    if (ctx_init(&c, A, o, plan, level_counts, lc_cap) != ORC_OK) return ORC_ERR_OOM;
    double *r = malloc(sizeof(double) * n), *p = malloc(sizeof(double) * n),
           *mu = malloc(sizeof(double) * n), *z = M ? malloc(sizeof(double) * n) : NULL;
    int st = ORC_OK;
    memset(info, 0, sizeof(*info));
    initial_residual(A, b, x, r);
    double nb = sqrt(orc_dot(b, b, n, plan));
    if (nb == 0.0) {
        for (int64_t i = 0; i < n; ++i) x[i] = 0.0;
        info->converged = 1; record(hist, hist_cap, 0, 0.0);
        goto done;
    }
    double rr = orc_dot(r, r, n, plan), rho;
    if (M) { ilu_apply(M, r, z); memcpy(p, z, sizeof(double) * n); rho = orc_dot(r, z, n, plan); }
    else   { memcpy(p, r, sizeof(double) * n); rho = rr; }
    ctx_set_tau(&c, M ? sqrt(orc_dot(p, p, n, plan)) : sqrt(rr));
    int64_t j = 0;
    for (;; ++j) {
        double relres = sqrt(rr) / nb;
        record(hist, hist_cap, j, relres);
        info->rel_residual = relres;
        if (relres < o->tol) { info->converged = 1; break; }
        if (j == o->max_iter) break;
        ctx_spmv(&c, p, mu);                                  /* mu = A~_j p_j */
        double sigma = orc_dot(mu, p, n, plan);               /* (mu, p_j) */
        if (!(sigma > 0.0) || !isfinite(sigma)) { st = ORC_ERR_BREAKDOWN; break; }
        double alpha = rho / sigma;
        for (int64_t i = 0; i < n; ++i) x[i] = fma(alpha, p[i], x[i]);
        for (int64_t i = 0; i < n; ++i) r[i] = fma(-alpha, mu[i], r[i]);
        rr = orc_dot(r, r, n, plan);
        double rho_new;
        if (M) { ilu_apply(M, r, z); rho_new = orc_dot(r, z, n, plan); }
        else rho_new = rr;
        double beta = rho_new / rho;
        rho = rho_new;
        const double* d = M ? z : r;
        for (int64_t i = 0; i < n; ++i) p[i] = fma(beta, p[i], d[i]);
    }
    info->iterations = j;
done:
    info->status = st; info->n_spmv = c.n_spmv;
    free(r); free(p); free(mu); free(z); ctx_free(&c);
    return st;
}

int orc_cg(const orc_tiles* A, const double* b, double* x, const orc_opts* o, const orc_plan* plan,
           double* hist, int64_t hist_cap, int64_t* level_counts, int64_t lc_cap, orc_info* info) {
    return orc_pcg(A, NULL, b, x, o, plan, hist, hist_cap, level_counts, lc_cap, info);
}

/* BiCGSTAB (and right-preconditioned PBiCGSTAB when M != NULL: phat = M^-1 p, shat = M^-1 s) */
int orc_pbicgstab(const orc_tiles* A, const orc_ilu* M, const double* b, double* x, const orc_opts* o,
                  const orc_plan* plan, double* hist, int64_t hist_cap, int64_t* level_counts,
                  int64_t lc_cap, orc_info* info) {
    int64_t n = A->n_rows;
    if (A->n_rows != A->n_cols) return ORC_ERR_INVALID_ARG;
    orc_ctx c;
    if (ctx_init(&c, A, o, plan, level_counts, lc_cap) != ORC_OK) return ORC_ERR_OOM;
    size_t nb8 = sizeof(double) * (size_t)n;
    double *r = malloc(nb8), *rh = malloc(nb8), *p = malloc(nb8), *mu = malloc(nb8),
           *s = malloc(nb8), *th = malloc(nb8);
    double *ph = M ? malloc(nb8) : NULL, *sh = M ? malloc(nb8) : NULL;
    int st = ORC_OK;
    memset(info, 0, sizeof(*info));
    initial_residual(A, b, x, r);
    double nb = sqrt(orc_dot(b, b, n, plan));
    if (nb == 0.0) {
        for (int64_t i = 0; i < n; ++i) x[i] = 0.0;
        info->converged = 1; record(hist, hist_cap, 0, 0.0);
        goto done;
    }
    memcpy(rh, r, nb8); memcpy(p, r, nb8);
    double rho = orc_dot(r, rh, n, plan);
    double rr = orc_dot(r, r, n, plan);
    if (M) { ilu_apply(M, p, ph); ctx_set_tau(&c, sqrt(orc_dot(ph, ph, n, plan))); }
    else ctx_set_tau(&c, sqrt(rr));
    int64_t j = 0;
    for (;; ++j) {
        double relres = sqrt(rr) / nb;
        record(hist, hist_cap, j, relres);
        info->rel_residual = relres;
        if (relres < o->tol) { info->converged = 1; break; }
        if (j == o->max_iter) break;
        if (M && j > 0) ilu_apply(M, p, ph);
        const double* pin = M ? ph : p;
        ctx_spmv(&c, pin, mu);                                /* mu = A~ p */
        double eta = orc_dot(mu, rh, n, plan);                /* (mu, r0*) */
        if (eta == 0.0 || !isfinite(eta)) { st = ORC_ERR_BREAKDOWN; break; }
        double alpha = rho / eta;
        for (int64_t i = 0; i < n; ++i) s[i] = fma(-alpha, mu[i], r[i]);   /* s = r - alpha mu */
        const double* sin_ = s;
        if (M) { ilu_apply(M, s, sh); sin_ = sh; }
        ctx_spmv(&c, sin_, th);                               /* theta = A~ s */
        double tt = orc_dot(th, th, n, plan);
        double ts = orc_dot(th, s, n, plan);
        if (tt == 0.0) {                                      /* theta == 0: take the half step */
            for (int64_t i = 0; i < n; ++i) x[i] = fma(alpha, pin[i], x[i]);
            memcpy(r, s, nb8);
            rr = orc_dot(r, r, n, plan);
            ++j;
            relres = sqrt(rr) / nb; record(hist, hist_cap, j, relres); info->rel_residual = relres;
            if (relres < o->tol) info->converged = 1; else st = ORC_ERR_BREAKDOWN;
            break;
        }
        double omega = ts / tt;
        if (omega == 0.0 || !isfinite(omega)) { st = ORC_ERR_BREAKDOWN; break; }
        for (int64_t i = 0; i < n; ++i) x[i] = fma(omega, sin_[i], fma(alpha, pin[i], x[i]));
        for (int64_t i = 0; i < n; ++i) r[i] = fma(-omega, th[i], s[i]);
        double rho_new = orc_dot(r, rh, n, plan);
        rr = orc_dot(r, r, n, plan);
        if (rho_new == 0.0 || !isfinite(rho_new)) {
            ++j; relres = sqrt(rr) / nb; record(hist, hist_cap, j, relres); info->rel_residual = relres;
            if (relres < o->tol) info->converged = 1; else st = ORC_ERR_BREAKDOWN;
            break;
        }
        double beta = (rho_new / rho) * (alpha / omega);
        rho = rho_new;
        for (int64_t i = 0; i < n; ++i) p[i] = fma(beta, fma(-omega, mu[i], p[i]), r[i]);
    }
    info->iterations = j;
done:
    info->status = st; info->n_spmv = c.n_spmv;
    free(r); free(rh); free(p); free(mu); free(s); free(th); free(ph); free(sh); ctx_free(&c);
    return st;
}

int orc_bicgstab(const orc_tiles* A, const double* b, double* x, const orc_opts* o, const orc_plan* plan,
                 double* hist, int64_t hist_cap, int64_t* level_counts, int64_t lc_cap, orc_info* info) {
    return orc_pbicgstab(A, NULL, b, x, o, plan, hist, hist_cap, level_counts, lc_cap, info);
}

/* textbook FP64 CG directly on CSR (Alg. 1), plain sequential dots: the CPU baseline and
 * an independent cross-check of the tiled path on exactly-representable matrices */
int orc_cg_csr(int64_t n, const int64_t* rowptr, const int32_t* colidx, const double* vals,
               const double* b, double* x, double tol, int64_t max_iter, double* hist, int64_t hist_cap,
               orc_info* info) {
    size_t nb8 = sizeof(double) * (size_t)n;
    double *r = malloc(nb8), *p = malloc(nb8), *mu = malloc(nb8);
    memset(info, 0, sizeof(*info));
    int st = ORC_OK;
    orc_spmv_csr(n, rowptr, colidx, vals, x, mu);
    for (int64_t i = 0; i < n; ++i) r[i] = b[i] - mu[i];
    if (all_zero(x, n)) memcpy(r, b, nb8);
    double nb = sqrt(orc_dot(b, b, n, NULL));
    double rho = orc_dot(r, r, n, NULL);
    memcpy(p, r, nb8);
    int64_t j = 0;
    if (nb == 0.0) { for (int64_t i = 0; i < n; ++i) x[i] = 0.0; info->converged = 1; goto done; }
    for (;; ++j) {
        double relres = sqrt(rho) / nb;
        record(hist, hist_cap, j, relres); info->rel_residual = relres;
        if (relres < tol) { info->converged = 1; break; }
        if (j == max_iter) break;
        orc_spmv_csr(n, rowptr, colidx, vals, p, mu);
        double sigma = orc_dot(mu, p, n, NULL);
        if (!(sigma > 0.0) || !isfinite(sigma)) { st = ORC_ERR_BREAKDOWN; break; }
        double alpha = rho / sigma;
        for (int64_t i = 0; i < n; ++i) x[i] = fma(alpha, p[i], x[i]);
        for (int64_t i = 0; i < n; ++i) r[i] = fma(-alpha, mu[i], r[i]);
        double rho_new = orc_dot(r, r, n, NULL);
        double beta = rho_new / rho;
        rho = rho_new;
        for (int64_t i = 0; i < n; ++i) p[i] = fma(beta, p[i], r[i]);
    }
    info->iterations = j;
done:
    info->status = st;
    free(r); free(p); free(mu);
    return st;
}

/* true relative residual ||b - A x|| / ||b|| on a CSR matrix (plain order) */
double orc_true_relres(int64_t n, const int64_t* rowptr, const int32_t* colidx, const double* vals,
                       const double* b, const double* x) {
    double* ax = malloc(sizeof(double) * (size_t)n);
    orc_spmv_csr(n, rowptr, colidx, vals, x, ax);
    double s = 0.0, sb = 0.0;
    for (int64_t i = 0; i < n; ++i) { double d = b[i] - ax[i]; s = fma(d, d, s); sb = fma(b[i], b[i], sb); }
    free(ax);
    return sqrt(s) / sqrt(sb);
}

/* ------------------------------------------------------------------------------------
 * 8. ILU(0) preconditioning ("incomplete LU factorization"; reading c-8 #20:
 *    ILU(0), FP64 factors).  IKJ variant on A's pattern (Saad, Alg. 10.4).
 *    L unit lower (strict lower part of lu), U upper including the diagonal.
 *    Forward  y_i = r_i - sum_{k<i} l_ik y_k      (fma chain, ascending k)
 *    Backward z_i = (y_i - sum_{k>i} u_ik z_k) / u_ii  (fma chain, descending k)
 *    Each chain runs in the order the substitution produces its unknowns (ascending for the
 *    forward solve, descending for the backward solve: the most recent unknown enters last);
 *    the paper fixes no order (reading R20).
 * ---------------------------------------------------------------------------------- */
int orc_ilu0(int64_t n, const int64_t* rowptr, const int32_t* colidx, const double* vals,
             double* lu, int64_t* diag) {
    int64_t nnz = rowptr[n];
    memcpy(lu, vals, sizeof(double) * (size_t)nnz);
    for (int64_t i = 0; i < n; ++i) {
        diag[i] = -1;
        for (int64_t k = rowptr[i]; k < rowptr[i + 1]; ++k) if (colidx[k] == i) diag[i] = k;
        if (diag[i] < 0) return ORC_ERR_ZERO_PIVOT;
    }
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t kk = rowptr[i]; kk < rowptr[i + 1] && colidx[kk] < i; ++kk) {
            int64_t k = colidx[kk];
            double akk = lu[diag[k]];
            if (akk == 0.0) return ORC_ERR_ZERO_PIVOT;
            lu[kk] = lu[kk] / akk;                                      /* a_ik = a_ik / a_kk */
            for (int64_t jj = kk + 1; jj < rowptr[i + 1]; ++jj) {       /* j > k in row i */
                int64_t jc = colidx[jj];
                for (int64_t m = diag[k] + 1; m < rowptr[k + 1]; ++m)   /* find a_kj in row k */
                    if (colidx[m] == jc) { lu[jj] = fma(-lu[kk], lu[m], lu[jj]); break; }
            }
        }
        if (lu[diag[i]] == 0.0) return ORC_ERR_ZERO_PIVOT;
    }
    return ORC_OK;
}

/* Recursive block SpTRSV ("we recursively divide a triangular matrix into two smaller
 * triangular blocks and one square block.  The SpTRSV operation is utilized for the triangular
 * blocks, and SpMV is applied to the square blocks"; the algorithm of [41]).  Readings (DESIGN.md
 * R27): a block of rows [lo, hi) with hi - lo >= 2 and depth > 0 splits at mid = lo + (hi - lo) / 2;
 * the square block's SpMV forms s_i = sum_k t_ik v_k over its columns (one fma chain from +0,
 * ascending k) and the right-hand side is then updated once, rhs_i = rhs_i - s_i; a leaf (depth 0
 * or fewer than 32 rows) is the row-by-row substitution restricted to the columns inside the leaf.
 * Split points are multiples of 16 (one tile row): mid = lo + 16 * floor((hi - lo) / 32).
 *
 * Lower (unit diagonal, the strict lower part of lu): rows [lo, hi), the contributions of the
 * columns < lo already subtracted from y[lo..hi) (y holds the right-hand side on entry).
 * Order: solve(lo, mid); square rows [mid, hi) x columns [lo, mid); solve(mid, hi). */
static int64_t rb_mid(int64_t lo, int64_t hi) { return lo + 16 * ((hi - lo) / 32); }
static void rb_lower(const orc_ilu* M, double* y, int64_t lo, int64_t hi, int depth) {
    if (depth == 0 || hi - lo < 32) {
        for (int64_t i = lo; i < hi; ++i) {
            double acc = y[i];
            for (int64_t k = M->rowptr[i]; k < M->diag[i]; ++k)
                if (M->colidx[k] >= lo) acc = fma(-M->lu[k], y[M->colidx[k]], acc);
            y[i] = acc;
        }
        return;
    }
    int64_t mid = rb_mid(lo, hi);
    rb_lower(M, y, lo, mid, depth - 1);
    for (int64_t i = mid; i < hi; ++i) {                 /* square block: SpMV, then the update */
        double s = 0.0;
        for (int64_t k = M->rowptr[i]; k < M->diag[i]; ++k) {
            int64_t c = M->colidx[k];
            if (c >= lo && c < mid) s = fma(M->lu[k], y[c], s);
        }
        y[i] = y[i] - s;
    }
    rb_lower(M, y, mid, hi, depth - 1);
}
/* Upper (diagonal u_ii in lu): rows [lo, hi), the contributions of the columns >= hi already
 * subtracted from z[lo..hi) (z holds the right-hand side on entry).  Order: solve(mid, hi);
 * square rows [lo, mid) x columns [mid, hi); solve(lo, mid).  Leaf rows descending. */
static void rb_upper(const orc_ilu* M, double* z, int64_t lo, int64_t hi, int depth) {
    if (depth == 0 || hi - lo < 32) {
        for (int64_t i = hi - 1; i >= lo; --i) {
            double acc = z[i];
            for (int64_t k = M->rowptr[i + 1] - 1; k > M->diag[i]; --k)
                if (M->colidx[k] < hi) acc = fma(-M->lu[k], z[M->colidx[k]], acc);
            z[i] = acc / M->lu[M->diag[i]];
        }
        return;
    }
    int64_t mid = rb_mid(lo, hi);
    rb_upper(M, z, mid, hi, depth - 1);
    for (int64_t i = lo; i < mid; ++i) {
        double s = 0.0;
        for (int64_t k = M->diag[i] + 1; k < M->rowptr[i + 1]; ++k) {
            int64_t c = M->colidx[k];
            if (c >= mid && c < hi) s = fma(M->lu[k], z[c], s);
        }
        z[i] = z[i] - s;
    }
    rb_upper(M, z, lo, mid, depth - 1);
}

static void ilu_apply(const orc_ilu* M, const double* r, double* z) {
    int64_t n = M->n;
    if (M->rb_depth > 0) {
        memcpy(z, r, sizeof(double) * (size_t)n);
        rb_lower(M, z, 0, n, M->rb_depth);
        rb_upper(M, z, 0, n, M->rb_depth);
        return;
    }
    double* y = malloc(sizeof(double) * (size_t)n);
    for (int64_t i = 0; i < n; ++i) {
        double acc = r[i];
        for (int64_t k = M->rowptr[i]; k < M->diag[i]; ++k) acc = fma(-M->lu[k], y[M->colidx[k]], acc);
        y[i] = acc;
    }
    for (int64_t i = n - 1; i >= 0; --i) {
        double acc = y[i];
        for (int64_t k = M->rowptr[i + 1] - 1; k > M->diag[i]; --k) acc = fma(-M->lu[k], z[M->colidx[k]], acc);
        z[i] = acc / M->lu[M->diag[i]];
    }
    free(y);
}

void orc_ilu_apply(const orc_ilu* M, const double* r, double* z) { ilu_apply(M, r, z); }

/* ------------------------------------------------------------------------------------
 * 9. The CPU baseline: textbook binary64 CSR CG / BiCGSTAB (Alg. 1-2,
 *    P:70) and their ILU(0)-preconditioned forms (PCG standard, PBiCGSTAB right-
 *    preconditioned as in orc_pcg / orc_pbicgstab), with the SpMV, the dots and the AXPYs
 *    spread over `threads` OpenMP threads (static schedule).  The dots are OpenMP sum
 *    reductions, so the summation order (not the arithmetic) differs from the sequential
 *    oracle; the triangular solves of the preconditioner stay sequential.  Pinned against the
 *    sequential oracle's FP64 mode (tests/test_oracle_baseline.py).
 * ---------------------------------------------------------------------------------- */
#ifdef _OPENMP
#include <omp.h>
#endif

static void par_spmv(int64_t n, const int64_t* rp, const int32_t* ci, const double* v, const double* x, double* y) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double acc = 0.0;
        for (int64_t k = rp[i]; k < rp[i + 1]; ++k) acc = fma(v[k], x[ci[k]], acc);
        y[i] = acc;
    }
}
static double par_dot(int64_t n, const double* u, const double* w) {
    double s = 0.0;
#pragma omp parallel for schedule(static) reduction(+ : s)
    for (int64_t i = 0; i < n; ++i) s = fma(u[i], w[i], s);
    return s;
}

int orc_baseline_threads(int threads) {
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
    return omp_get_max_threads();
#else
    (void)threads;
    return 1;
#endif
}

/* CG (M == NULL) or PCG with ILU(0) */
int orc_cg_csr_omp(int64_t n, const int64_t* rp, const int32_t* ci, const double* v, const orc_ilu* M,
                   const double* b, double* x, double tol, int64_t max_iter, orc_info* info) {
    size_t nb8 = sizeof(double) * (size_t)(n > 0 ? n : 1);
    double *r = malloc(nb8), *p = malloc(nb8), *mu = malloc(nb8), *z = M ? malloc(nb8) : NULL;
    memset(info, 0, sizeof(*info));
    int st = ORC_OK;
    par_spmv(n, rp, ci, v, x, mu);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) r[i] = b[i] - mu[i];
    double nb = sqrt(par_dot(n, b, b));
    double rr = par_dot(n, r, r), rho;
    int64_t j = 0;
    if (nb == 0.0) { for (int64_t i = 0; i < n; ++i) x[i] = 0.0; info->converged = 1; goto done; }
    if (M) { ilu_apply(M, r, z); memcpy(p, z, nb8); rho = par_dot(n, r, z); }
    else { memcpy(p, r, nb8); rho = rr; }
    for (;; ++j) {
        double relres = sqrt(rr) / nb;
        info->rel_residual = relres;
        if (relres < tol) { info->converged = 1; break; }
        if (j == max_iter) break;
        par_spmv(n, rp, ci, v, p, mu);
        double sigma = par_dot(n, mu, p);
        if (!(sigma > 0.0) || !isfinite(sigma)) { st = ORC_ERR_BREAKDOWN; break; }
        double alpha = rho / sigma;
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) { x[i] = fma(alpha, p[i], x[i]); r[i] = fma(-alpha, mu[i], r[i]); }
        rr = par_dot(n, r, r);
        double rho_new;
        if (M) { ilu_apply(M, r, z); rho_new = par_dot(n, r, z); } else rho_new = rr;
        double beta = rho_new / rho;
        rho = rho_new;
        const double* d = M ? z : r;
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) p[i] = fma(beta, p[i], d[i]);
    }
done:
    info->iterations = j; info->status = st; info->n_spmv = j;
    free(r); free(p); free(mu); free(z);
    return st;
}

/* BiCGSTAB (M == NULL) or right-preconditioned PBiCGSTAB with ILU(0) */
int orc_bicgstab_csr_omp(int64_t n, const int64_t* rp, const int32_t* ci, const double* v, const orc_ilu* M,
                         const double* b, double* x, double tol, int64_t max_iter, orc_info* info) {
    size_t nb8 = sizeof(double) * (size_t)(n > 0 ? n : 1);
    double *r = malloc(nb8), *rh = malloc(nb8), *p = malloc(nb8), *mu = malloc(nb8), *s = malloc(nb8), *th = malloc(nb8);
    double *ph = M ? malloc(nb8) : NULL, *sh = M ? malloc(nb8) : NULL;
    memset(info, 0, sizeof(*info));
    int st = ORC_OK;
    int64_t j = 0;
    par_spmv(n, rp, ci, v, x, mu);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) r[i] = b[i] - mu[i];
    double nb = sqrt(par_dot(n, b, b));
    if (nb == 0.0) { for (int64_t i = 0; i < n; ++i) x[i] = 0.0; info->converged = 1; goto done; }
    memcpy(rh, r, nb8); memcpy(p, r, nb8);
    double rho = par_dot(n, r, rh), rr = par_dot(n, r, r);
    for (;; ++j) {
        double relres = sqrt(rr) / nb;
        info->rel_residual = relres;
        if (relres < tol) { info->converged = 1; break; }
        if (j == max_iter) break;
        const double* pin = p;
        if (M) { ilu_apply(M, p, ph); pin = ph; }
        par_spmv(n, rp, ci, v, pin, mu);
        double eta = par_dot(n, mu, rh);
        if (eta == 0.0 || !isfinite(eta)) { st = ORC_ERR_BREAKDOWN; break; }
        double alpha = rho / eta;
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) s[i] = fma(-alpha, mu[i], r[i]);
        const double* sin_ = s;
        if (M) { ilu_apply(M, s, sh); sin_ = sh; }
        par_spmv(n, rp, ci, v, sin_, th);
        double tt = par_dot(n, th, th), ts = par_dot(n, th, s);
        if (tt == 0.0) {
#pragma omp parallel for schedule(static)
            for (int64_t i = 0; i < n; ++i) { x[i] = fma(alpha, pin[i], x[i]); r[i] = s[i]; }
            rr = par_dot(n, r, r); ++j;
            info->rel_residual = sqrt(rr) / nb;
            if (info->rel_residual < tol) info->converged = 1; else st = ORC_ERR_BREAKDOWN;
            break;
        }
        double omega = ts / tt;
        if (omega == 0.0 || !isfinite(omega)) { st = ORC_ERR_BREAKDOWN; break; }
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) { x[i] = fma(omega, sin_[i], fma(alpha, pin[i], x[i])); r[i] = fma(-omega, th[i], s[i]); }
        double rho_new = par_dot(n, r, rh);
        rr = par_dot(n, r, r);
        if (rho_new == 0.0 || !isfinite(rho_new)) {
            ++j; info->rel_residual = sqrt(rr) / nb;
            if (info->rel_residual < tol) info->converged = 1; else st = ORC_ERR_BREAKDOWN;
            break;
        }
        double beta = (rho_new / rho) * (alpha / omega);
        rho = rho_new;
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; ++i) p[i] = fma(beta, fma(-omega, mu[i], p[i]), r[i]);
    }
done:
    info->iterations = j; info->status = st; info->n_spmv = 2 * j;
    free(r); free(rh); free(p); free(mu); free(s); free(th); free(ph); free(sh);
    return st;
}

/* ------------------------------------------------------------------------------------
 * 10. Single-reduction CG (the one-barrier variant of Alg. 1; Chronopoulos &
 *     Gear, "s-step iterative methods", 1989): the two dots of an iteration share ONE reduction
 *     because delta = (A r, r) replaces (A p, p):
 *       r0 = b - A~ x0 ; w0 = A~_0 r0 ; gamma0 = (r0, r0) ; delta0 = (w0, r0) ; alpha0 = gamma0/delta0
 *       beta0 = 0 ; p = s = 0
 *       loop i: relres_i = sqrt(gamma_i)/||b|| ; stop test as in CG
 *         p = fma(beta_i, p, r) ; s = fma(beta_i, s, w)          (s = A~ p by recurrence)
 *         x = fma(alpha_i, p, x) ; r = fma(-alpha_i, s, r)
 *         w = A~_{i+1} r                                        (the SpMV input is r: the dynamic
 *                                                                switch watches r)
 *         gamma' = (r, r) ; delta' = (w, r)                     (one reduction)
 *         beta' = gamma'/gamma ; t = (beta' * gamma') / alpha ; alpha' = gamma' / (delta' - t)
 *       breakdown: delta' - t <= 0 or non-finite (SPD => (p', A p') > 0).
 *     Iterations = loop passes (the SpMVs are iterations + 1).  tau from ||r0|| (v0 = r0).
 * ---------------------------------------------------------------------------------- */
int orc_cg_single_reduction(const orc_tiles* A, const double* b, double* x, const orc_opts* o, const orc_plan* plan,
                            double* hist, int64_t hist_cap, int64_t* level_counts, int64_t lc_cap, orc_info* info) {
    int64_t n = A->n_rows;
    if (A->n_rows != A->n_cols) return ORC_ERR_INVALID_ARG;
    orc_ctx c;
    if (ctx_init(&c, A, o, plan, level_counts, lc_cap) != ORC_OK) return ORC_ERR_OOM;
    size_t nb8 = sizeof(double) * (size_t)(n > 0 ? n : 1);
    double *r = malloc(nb8), *p = calloc((size_t)(n > 0 ? n : 1), sizeof(double)), *s = calloc((size_t)(n > 0 ? n : 1), sizeof(double)),
           *w = malloc(nb8);
    int st = ORC_OK;
    int64_t j = 0;
    memset(info, 0, sizeof(*info));
    initial_residual(A, b, x, r);
    double nb = sqrt(orc_dot(b, b, n, plan));
    if (nb == 0.0) {
        for (int64_t i = 0; i < n; ++i) x[i] = 0.0;
        info->converged = 1; record(hist, hist_cap, 0, 0.0);
        goto done;
    }
    double gamma = orc_dot(r, r, n, plan);
    ctx_set_tau(&c, sqrt(gamma));
    double alpha = 0.0, beta = 0.0;
    {
        double relres = sqrt(gamma) / nb;
        if (!(relres < o->tol) && o->max_iter > 0) {      /* the first SpMV only when iterating */
            ctx_spmv(&c, r, w);
            double delta = orc_dot(w, r, n, plan);
            if (!(delta > 0.0) || !isfinite(delta)) { st = ORC_ERR_BREAKDOWN; record(hist, hist_cap, 0, relres); info->rel_residual = relres; goto done; }
            alpha = gamma / delta;
        }
    }
    for (;; ++j) {
        double relres = sqrt(gamma) / nb;
        record(hist, hist_cap, j, relres);
        info->rel_residual = relres;
        if (relres < o->tol) { info->converged = 1; break; }
        if (j == o->max_iter) break;
        for (int64_t i = 0; i < n; ++i) {
            p[i] = fma(beta, p[i], r[i]);
            s[i] = fma(beta, s[i], w[i]);
            x[i] = fma(alpha, p[i], x[i]);
            r[i] = fma(-alpha, s[i], r[i]);
        }
        ctx_spmv(&c, r, w);
        double gamma1 = orc_dot(r, r, n, plan);
        double delta1 = orc_dot(w, r, n, plan);
        double beta1 = gamma1 / gamma;
        double t = (beta1 * gamma1) / alpha;
        double den = delta1 - t;
        if (!(den > 0.0) || !isfinite(den)) {
            /* the residual is updated: report it before breaking down */
            ++j; relres = sqrt(gamma1) / nb; record(hist, hist_cap, j, relres); info->rel_residual = relres;
            if (relres < o->tol) info->converged = 1; else st = ORC_ERR_BREAKDOWN;
            break;
        }
        alpha = gamma1 / den;
        beta = beta1;
        gamma = gamma1;
    }
done:
    info->iterations = j; info->status = st; info->n_spmv = c.n_spmv;
    free(r); free(p); free(s); free(w); ctx_free(&c);
    return st;
}
