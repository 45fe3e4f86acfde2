// kernels.cuh -- device building blocks shared by the persistent solver kernels and the
// standalone mf_spmv / mf_levels / mf_dot kernels.
//
//  * spmv_tile_row: Alg. 5 for one tile row, one half-warp, lane r = row 16*TR+r.
//    Each row is ONE fma chain over its nonzeros in ascending column order (the slice layout
//    stores them in that order), so no floating-point atomics are needed (Alg. 5 l.13's
//    atomicAdd disappears) and the result is bit-identical for any launch shape.
//  * level_of / tile_code: Alg. 4 thresholds and the effective precision e_t.
//  * Reductions: the fixed tree of DESIGN.md "Reduction order" (thread fma chain -> warp
//    xor-butterfly -> tree32 over warps -> tree32 over CTAs).
#pragma once

#include "mf_internal.cuh"

namespace mfk {

constexpr int STAGE = 32;          // tile codes staged in smem per half-warp
constexpr int BYP = 4;

struct Mat {
    int64_t n_rows, n_cols, ntr;
    const int64_t* __restrict__ tr_slot;
    const int64_t* __restrict__ tr_tile;
    const uint32_t* __restrict__ tile_info;
    const uint16_t* __restrict__ sidx;
    const double* __restrict__ p64;
    const float* __restrict__ p32;
    const __half* __restrict__ p16;
    const uint8_t* __restrict__ p8;
};

__device__ __forceinline__ unsigned hw_mask() { return (threadIdx.x & 16) ? 0xFFFF0000u : 0x0000FFFFu; }

__device__ __forceinline__ int hw_min_i(int v, unsigned m) {
    for (int o = 8; o >= 1; o >>= 1) v = min(v, __shfl_xor_sync(m, v, o));
    return v;
}

// (tile column << 3) | e_t.   e_t = bypass | max_prec(floor, min_prec(TilePrec, level))
template <bool DYN>
__device__ __forceinline__ uint32_t tile_code(uint32_t info, const uint8_t* __restrict__ level, int range_guard) {
    const uint32_t tc = info >> 4;
    int e = (int)(info & 3u);
    if (DYN) {
        const int lv = level[tc];
        if (lv == BYP) return (tc << 3) | BYP;
        e = max(e, lv);
        if (range_guard) e = min(e, (int)((info >> 2) & 3u));
    }
    return (tc << 3) | (uint32_t)e;
}

__device__ __forceinline__ double load_val(const Mat& A, int e, int64_t pos) {
    if (e == 0) return A.p64[pos];
    if (e == 1) return (double)A.p32[pos];
    if (e == 2) return f16_to_d(A.p16[pos]);
    return e4m3_to_d(A.p8[pos]);
}

// Per-thread tile / nonzero counters by effective precision (FP64..FP8, bypass), packed in
// 21-bit fields so that a data-dependent index never turns into local-memory traffic.
struct Counts {
    unsigned long long t_lo, t_hi, n_lo, n_hi;
    __device__ __forceinline__ void zero() { t_lo = t_hi = n_lo = n_hi = 0; }
    __device__ __forceinline__ static void bump(unsigned long long& lo, unsigned long long& hi, int e) {
        if (e < 3) lo += 1ull << (21 * e); else hi += 1ull << (21 * (e - 3));
    }
    __device__ __forceinline__ void tile(int e) { bump(t_lo, t_hi, e); }
    __device__ __forceinline__ void nz(int e) { bump(n_lo, n_hi, e); }
    __device__ __forceinline__ static int field(unsigned long long lo, unsigned long long hi, int q) {
        return (int)(((q < 3 ? lo : hi) >> (21 * (q < 3 ? q : q - 3))) & 0x1FFFFFull);
    }
    __device__ __forceinline__ int tiles(int q) const { return field(t_lo, t_hi, q); }
    __device__ __forceinline__ int nnz(int q) const { return field(n_lo, n_hi, q); }
};

// mu_row = (A~ x)_row for row 16*TR + lane.  stage: this half-warp's STAGE-entry smem slab.
template <bool DYN, bool COUNT>
__device__ __forceinline__ double spmv_tile_row(const Mat& A, int64_t TR, int lane, const double* x,
                                                const uint8_t* __restrict__ level, int range_guard,
                                                uint32_t* stage, unsigned m, Counts* cnt) {
    const int64_t tb = A.tr_tile[TR];
    const int nt = (int)(A.tr_tile[TR + 1] - tb);
    const int64_t sb = A.tr_slot[TR];
    const int W = (int)(A.tr_slot[TR + 1] - sb);
    const bool staged = nt <= STAGE;
    __syncwarp(m);
    for (int jj = lane; jj < nt; jj += 16) {
        const uint32_t code = tile_code<DYN>(A.tile_info[tb + jj], level, range_guard);
        if (staged) stage[jj] = code;
        if (COUNT) cnt->tile((int)(code & 7u));
    }
    __syncwarp(m);
    double acc = 0.0;
    const uint16_t* __restrict__ sp = A.sidx + sb * 16 + lane;
    const int64_t pbase = sb * 16 + lane;
    int k = 0;
#define MF_SLOT_DECODE(S, CODE, E, COL)                                                   \
    uint32_t CODE = 0; int E = BYP; int64_t COL = 0;                                       \
    if (S != mf::SLOT_PAD) {                                                               \
        const int j_ = S >> 4;                                                             \
        CODE = staged ? stage[j_] : tile_code<DYN>(A.tile_info[tb + j_], level, range_guard); \
        E = (int)(CODE & 7u);                                                              \
        COL = (int64_t)(CODE >> 3) * 16 + (S & 15);                                        \
        if (COUNT) cnt->nz(E);                                                          \
    }
    for (; k + 4 <= W; k += 4) {
        const uint16_t s0 = sp[(k + 0) * 16], s1 = sp[(k + 1) * 16], s2 = sp[(k + 2) * 16], s3 = sp[(k + 3) * 16];
        MF_SLOT_DECODE(s0, c0, e0, col0)
        MF_SLOT_DECODE(s1, c1, e1, col1)
        MF_SLOT_DECODE(s2, c2, e2, col2)
        MF_SLOT_DECODE(s3, c3, e3, col3)
        double v0 = 0, v1 = 0, v2 = 0, v3 = 0, x0 = 0, x1 = 0, x2 = 0, x3 = 0;
        if (e0 != BYP) { v0 = load_val(A, e0, pbase + (k + 0) * 16); x0 = x[col0]; }
        if (e1 != BYP) { v1 = load_val(A, e1, pbase + (k + 1) * 16); x1 = x[col1]; }
        if (e2 != BYP) { v2 = load_val(A, e2, pbase + (k + 2) * 16); x2 = x[col2]; }
        if (e3 != BYP) { v3 = load_val(A, e3, pbase + (k + 3) * 16); x3 = x[col3]; }
        if (e0 != BYP) acc = __fma_rn(v0, x0, acc);
        if (e1 != BYP) acc = __fma_rn(v1, x1, acc);
        if (e2 != BYP) acc = __fma_rn(v2, x2, acc);
        if (e3 != BYP) acc = __fma_rn(v3, x3, acc);
    }
    for (; k < W; ++k) {
        const uint16_t s0 = sp[k * 16];
        MF_SLOT_DECODE(s0, c0, e0, col0)
        if (e0 != BYP) acc = __fma_rn(load_val(A, e0, pbase + k * 16), x[col0], acc);
    }
#undef MF_SLOT_DECODE
    return acc;
}

// Alg. 4 with the P:174 intervals (reading R5) on |v| (R7); NaN -> FP64.
struct Thresh {
    double t0, t1, t2, t3;
};
__device__ __forceinline__ int level_of(double v, const Thresh& th) {
    const double a = fabs(v);
    if (a < th.t0) return 4;
    if (a < th.t1) return 3;
    if (a < th.t2) return 2;
    if (a < th.t3) return 1;
    return 0;   // includes NaN
}

// ---- reductions
__device__ __forceinline__ double butterfly32(double v) {
    for (int o = 16; o >= 1; o >>= 1) v = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
// lane l: s = +0; s += x[l], x[l+32], ...; then butterfly.  Called by a full warp.
__device__ __forceinline__ double tree32(const double* x, int c) {
    const int l = threadIdx.x & 31;
    double s = 0.0;
    for (int i = l; i < c; i += 32) s = __dadd_rn(s, x[i]);
    return butterfly32(s);
}

}  // namespace mfk
