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
    const uint16_t* __restrict__ sidx;    // compact layout
    const uint8_t* __restrict__ sslot;    // tile-synchronous layout
    const uint32_t* __restrict__ colw;    // tile-synchronous layout
    int ts;
    int max_w;                            // widest tile-row slice (slice columns)
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

// ------------------------------------------------------------------------------------------
// Windowed SpMV over the contiguous tile rows [tr0, tr1) of one CTA (all B threads call it).
// A window is up to WIN_TR tile rows (a multiple of H = B/16 so that half-warp h always gets
// tile rows tr0 + h + kH, the row mapping of the dot-product contract).  Per window the CTA
// stages in shared memory, with coalesced (cp.async) copies:
//   compact layout:          the tile codes (tile column + e_t) of the window's tiles;
//   tile-synchronous layout: the slot bytes and the per-column tile words of the window's
//                            slice columns (static), plus, once per SpMV, the level bytes of
//                            the column segments the CTA gathers.
// Each half-warp then needs one global round trip per chunk of slots (values and x).
constexpr int WIN_TR = 1024;
constexpr int CODE_CAP = 8192;
constexpr int COL_CAP = 2048;
constexpr int LEV_CAP = 16384;
constexpr int WIN_BUF_BYTES = (COL_CAP * 16 + COL_CAP * 4 + LEV_CAP) > CODE_CAP * 4 ? (COL_CAP * 16 + COL_CAP * 4 + LEV_CAP)
                                                                                      : CODE_CAP * 4;

struct WinSmem {
    int32_t* hs;     // [WIN_TR+1] slot (slice column) offset of each tile row, relative to s0
    int32_t* ht;     // [WIN_TR+1] tile offset, relative to t0
    int64_t* misc;   // [4]: -, -, window end, staged
    unsigned long long* pb;   // [4] value-plane base addresses (FP64, FP32, FP16, E4M3)
    unsigned char* buf;   // [WIN_BUF_BYTES]: compact: uint32 code[CODE_CAP]
                          //                  TS: uint8 ss[COL_CAP*16] | uint32 cw[COL_CAP] | uint8 lev[LEV_CAP]
};
constexpr size_t WIN_SMEM_BYTES = 2 * (WIN_TR + 1) * 4 + 4 * 8 + 8 + 4 * 8 + WIN_BUF_BYTES + 16;

// Value fetch: ONE aligned 8-byte load from plane[e] + pos*size(e) (planes are 8-byte aligned and
// padded), the needed bytes shifted down.  The 8-byte word lies in the same 32-byte DRAM sector
// as the value, so this moves no extra HBM bytes; it replaces four predicated loads.
__device__ __forceinline__ uint64_t load_raw(const unsigned long long* pbase, int e, int64_t pos) {
    const unsigned long long a = pbase[e] + ((unsigned long long)pos << (3 - e));
    const unsigned long long w = __ldg(reinterpret_cast<const unsigned long long*>(a & ~7ull));
    return w >> ((a & 7ull) * 8);
}
// exact upcast of the stored bits at precision e (0 FP64, 1 FP32, 2 FP16, 3 E4M3) to binary64
__device__ __forceinline__ double decode_val(int e, uint64_t raw) {
    const uint32_t lo = (uint32_t)raw;
    const __half_raw h8 = __nv_cvt_fp8_to_halfraw((__nv_fp8_storage_t)(lo & 0xFFu), __NV_E4M3);
    const unsigned short hb = e == 3 ? h8.x : (unsigned short)lo;
    const float f16 = __half2float(__ushort_as_half(hb));
    const float f = e >= 2 ? f16 : __uint_as_float(lo);
    const double d = (double)f;
    return e == 0 ? __longlong_as_double((long long)raw) : d;
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// compact layout: process slot words s[0..cnt) of one lane; returns updated acc
template <bool DYN, bool COUNT, int N>
__device__ __forceinline__ double slot_block(const Mat& A, const unsigned long long* w_pb, const uint16_t (&s)[N], int cnt, int64_t pos0,
                                             const uint32_t* code, bool staged, int64_t tb_abs,
                                             const uint8_t* __restrict__ level, int range_guard,
                                             const double* x, double acc, Counts* cntp) {
    uint64_t raw[N];
    double xv[N];
    int ev[N];
#pragma unroll
    for (int q = 0; q < N; ++q) {
        ev[q] = BYP;
        raw[q] = 0;
        xv[q] = 0.0;
        if (q < cnt && s[q] != mf::SLOT_PAD) {
            const int j = s[q] >> 4;
            const uint32_t c = staged ? code[j] : tile_code<DYN>(A.tile_info[tb_abs + j], level, range_guard);
            ev[q] = (int)(c & 7u);
            if (COUNT) cntp->nz(ev[q]);
            if (ev[q] != BYP) {
                raw[q] = load_raw(w_pb, ev[q], pos0 + q * 16);
                xv[q] = x[(int64_t)(c >> 3) * 16 + (s[q] & 15)];
            }
        }
    }
#pragma unroll
    for (int q = 0; q < N; ++q)
        if (ev[q] != BYP) acc = __fma_rn(decode_val(ev[q], raw[q]), xv[q], acc);
    return acc;
}

// e_t of a tile-synchronous column word (same rule as tile_code)
template <bool DYN>
__device__ __forceinline__ uint32_t col_code(uint32_t word, const uint8_t* lev_s, int32_t seg_lo, bool lev_staged,
                                             const uint8_t* __restrict__ level, int range_guard) {
    const uint32_t tc = word >> 4;
    int e = (int)(word & 3u);
    if (DYN) {
        const int lv = lev_staged ? lev_s[tc - seg_lo] : level[tc];
        if (lv == BYP) return (tc << 3) | BYP;
        e = max(e, lv);
        if (range_guard) e = min(e, (int)((word >> 2) & 3u));
    }
    return (tc << 3) | (uint32_t)e;
}

// tile-synchronous layout: columns of one tile row; ss = slot bytes, cd = column codes
// (tile column << 3 | e_t, uniform across the 16 lanes)
template <bool COUNT, int N>
__device__ __forceinline__ double ts_block(const Mat& A, const unsigned long long* w_pb, const uint8_t* ss, const uint32_t* cd, int cnt, int lane,
                                           int64_t pos0, const double* x, double acc, Counts* cntp) {
    uint64_t raw[N];
    double xv[N];
    int ev[N];
#pragma unroll
    for (int q = 0; q < N; ++q) {
        const uint32_t lc = q < cnt ? ss[q * 16 + lane] : 0xFFu;
        const uint32_t c = q < cnt ? cd[q] : (uint32_t)BYP;
        ev[q] = lc == 0xFFu ? BYP : (int)(c & 7u);
        if (COUNT && lc != 0xFFu) cntp->nz(ev[q]);
        raw[q] = 0;
        xv[q] = 0.0;
        if (ev[q] != BYP) {
            raw[q] = load_raw(w_pb, ev[q], pos0 + q * 16);
            xv[q] = x[(int64_t)(c >> 3) * 16 + lc];
        }
    }
#pragma unroll
    for (int q = 0; q < N; ++q)
        if (ev[q] != BYP) acc = __fma_rn(decode_val(ev[q], raw[q]), xv[q], acc);
    return acc;
}

// ------------------------------------------------------------------------------------------
// Tile-synchronous SpMV, software-pipelined over windows of 2H tile rows (half-warp h owns tile
// rows w0+h and w0+H+h of each window -- the dot-contract mapping tr0 + h + kH).
// Staging of window k+1 overlaps the compute of window k:
//   * slot bytes: cp.async (16 B per slice column) into the other smem stage;
//   * per-column records {value pointer at e_t, x offset, e_t}: column words prefetched into
//     registers before computing window k, turned into records after it.
// The consumer issues every load of a tile row at once (values: one aligned 8-byte word each; x:
// one 8-byte load each), then runs the fma chain.  A bypassed / padding slot contributes
// fma(0, 0, acc) == acc exactly (acc starts at +0 and can never become -0).
constexpr int TSP_COLS = 1024;   // slice columns per window (cap)
constexpr int TSP_CPT = 2;       // column words prefetched per thread (TSP_COLS / B for B = 512)
constexpr int TSP_Q = 9;         // columns per load batch of one tile row
struct TsRec {
    unsigned long long vptr;     // plane_e + column slot base * size(e)   (0: bypassed column)
    int32_t xoff;                // tile column * 16
    int32_t e;                   // e_t
};
constexpr size_t TSP_STAGE_BYTES = (size_t)TSP_COLS * 16 + (size_t)TSP_COLS * sizeof(TsRec);
constexpr size_t TSP_SMEM_BYTES = 2 * ((size_t)TSP_COLS * sizeof(TsRec) + (size_t)TSP_COLS * 16 + (((2 * 512 + 1) * 4 + 15) / 16 * 16)) + LEV_CAP + 64;
constexpr size_t SPMV_SMEM_BYTES = TSP_SMEM_BYTES > WIN_SMEM_BYTES ? TSP_SMEM_BYTES : WIN_SMEM_BYTES;

// the two SpMV scratch views over one shared-memory region (a matrix uses one layout)
__device__ __forceinline__ void carve_spmv(unsigned char* p, WinSmem& w, struct TsSmem& ts);

// stage st occupies [base + st*TSP_STRIDE, ...): records | slot bytes | headers; then the levels.
// (Stage pointers are computed, not looked up: a runtime-indexed pointer array would live in
// local memory.)
constexpr size_t TSP_HS_BYTES = ((2 * 512 + 1) * 4 + 15) / 16 * 16;
constexpr size_t TSP_STRIDE = (size_t)TSP_COLS * sizeof(TsRec) + (size_t)TSP_COLS * 16 + TSP_HS_BYTES;
struct TsSmem {
    unsigned char* base;
    __device__ __forceinline__ TsRec* rec(int st) const { return reinterpret_cast<TsRec*>(base + st * TSP_STRIDE); }
    __device__ __forceinline__ uint8_t* ss(int st) const { return base + st * TSP_STRIDE + (size_t)TSP_COLS * sizeof(TsRec); }
    __device__ __forceinline__ int32_t* hs(int st) const {
        return reinterpret_cast<int32_t*>(base + st * TSP_STRIDE + (size_t)TSP_COLS * sizeof(TsRec) + (size_t)TSP_COLS * 16);
    }
    __device__ __forceinline__ uint8_t* lev() const { return base + 2 * TSP_STRIDE; }
};

__device__ __forceinline__ uint32_t lds_u8(const void* p) {
    uint32_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(p)));
    return v;
}
__device__ __forceinline__ void lds_rec(const void* p, unsigned long long& vptr, int& xoff, int& e) {
    unsigned lo, hi, xo, ee;
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(lo), "=r"(hi), "=r"(xo), "=r"(ee) : "r"((unsigned)__cvta_generic_to_shared(p)));
    vptr = ((unsigned long long)hi << 32) | lo;
    xoff = (int)xo;
    e = (int)ee;
}

// one tile row of a window: all its slots' loads are issued before the fma chain.  Padding and
// bypassed slots load a zero value word (their x load reads a valid element of the same
// segment), so every slot is one unconditional fma: fma(0, x, acc) == acc exactly.
template <bool COUNT>
__device__ __forceinline__ double ts_row(const uint8_t* ss, const TsRec* rec, int a, int W, int lane,
                                         const double* x, Counts* cntp) {
    double acc = 0.0;
    for (int k = 0; k < W; k += TSP_Q) {
        unsigned long long wv[TSP_Q];
        double xv[TSP_Q];
        uint32_t meta[TSP_Q];          // ((addr & 7) << 11) | e
        const int n = W - k;
#pragma unroll
        for (int q = 0; q < TSP_Q; ++q) {
            // columns past the tile row (q >= n) read column a (always staged) and are masked
            const bool in = q < n;
            const int c = in ? a + k + q : a;
            const uint32_t lc = lds_u8(ss + c * 16 + lane);
            unsigned long long vptr;
            int xoff, e;
            lds_rec(rec + c, vptr, xoff, e);
            if (COUNT && in && lc != 0xFFu) cntp->nz(e);
            const bool ok = in && lc != 0xFFu && e != BYP;
            const unsigned long long ad = vptr + ((unsigned long long)lane << (3 - (e & 3)));
            meta[q] = ((uint32_t)(ad & 7ull) << 11) | (uint32_t)(e & 3);
            unsigned long long w = 0ull;
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.global.nc.u64 %0, [%1];\n\t}"
                         : "+l"(w) : "l"(ad & ~7ull), "r"((unsigned)ok));
            wv[q] = w;
            xv[q] = x[xoff + (int)(lc & 15u)];
        }
#pragma unroll
        for (int q = 0; q < TSP_Q; ++q)
            acc = __fma_rn(decode_val((int)(meta[q] & 3u), wv[q] >> (meta[q] >> 8)), xv[q], acc);
    }
    return acc;
}

template <bool DYN, bool COUNT, class Emit>
__device__ __forceinline__ void spmv_ts_pipe(const Mat& A, int64_t tr0, int64_t tr1, const double* x, const uint8_t* __restrict__ level,
                             int range_guard, const TsSmem& sm, Counts* cnt, int32_t seg_lo, int32_t seg_hi, Emit emit) {
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
    const int NW = 2 * H;                       // tile rows per window
    const int32_t nlev = seg_hi - seg_lo + 1;
    const bool lev_staged = DYN && nlev > 0 && nlev <= LEV_CAP;
    const unsigned long long pb0 = (unsigned long long)A.p64, pb1 = (unsigned long long)A.p32,
                             pb2 = (unsigned long long)A.p16, pb3 = (unsigned long long)A.p8;
    __syncthreads();
    if (lev_staged)
        for (int i = t; i < nlev; i += B) sm.lev()[i] = level[seg_lo + i];
    if (COUNT)
        for (int64_t i = A.tr_tile[tr0] + t; i < A.tr_tile[tr1]; i += B)
            cnt->tile(tile_code<DYN>(A.tile_info[i], level, range_guard) & 7u);
    // prefetch state for the next window: header (thread i <= NW) and column words (registers)
    uint32_t cw0 = 0u, cw1 = 0u;
    static_assert(TSP_CPT == 2, "two column words per thread");
#define TSP_FETCH_HDR(W0, HDR)                                                               \
    {                                                                                       \
        const int64_t nw_ = min((int64_t)NW, tr1 - (W0));                                   \
        HDR = t <= nw_ ? A.tr_slot[(W0) + t] : A.tr_slot[(W0) + nw_];                       \
    }
#define TSP_PUBLISH_HDR(ST, W0, HDR)                                                         \
    {                                                                                       \
        const int64_t nw_ = min((int64_t)NW, tr1 - (W0));                                   \
        if (t <= nw_) sm.hs(ST)[t] = (int32_t)((HDR) - A.tr_slot[W0]);                      \
    }
#define TSP_ISSUE(ST, SBASE, NCOL)                                                           \
    {                                                                                       \
        for (int c_ = t; c_ < (NCOL); c_ += B) cp_async16(sm.ss(ST) + c_ * 16, A.sslot + ((SBASE) + c_) * 16); \
        cw0 = t < (NCOL) ? __ldg(A.colw + (SBASE) + t) : 0u;                                \
        cw1 = t + B < (NCOL) ? __ldg(A.colw + (SBASE) + t + B) : 0u;                        \
    }
    auto build_rec = [&](int st, int64_t sbase, int c, uint32_t word) {
        const uint32_t tc = word >> 4;
        int e = (int)(word & 3u);
        if (DYN) {
            const int lv = lev_staged ? sm.lev()[tc - seg_lo] : level[tc];
            if (lv == BYP) e = BYP;
            else {
                e = max(e, lv);
                if (range_guard) e = min(e, (int)((word >> 2) & 3u));
            }
        }
        const unsigned long long pbase = e == 0 ? pb0 : e == 1 ? pb1 : e == 2 ? pb2 : pb3;
        const unsigned long long vptr = pbase + ((unsigned long long)((sbase + c) * 16) << (3 - (e & 3)));
        sm.rec(st)[c] = TsRec{e == BYP ? 0ull : vptr, (int32_t)(tc * 16), e};
    };
#define TSP_BUILD(ST, SBASE, NCOL)                                                           \
    {                                                                                       \
        if (t < (NCOL)) build_rec(ST, SBASE, t, cw0);                                       \
        if (t + B < (NCOL)) build_rec(ST, SBASE, t + B, cw1);                               \
    }
    // window 0: staged synchronously
    int64_t w0 = tr0;
    int stage = 0;
    int64_t hdr = 0;
    if (w0 < tr1) TSP_FETCH_HDR(w0, hdr)
    __syncthreads();
    if (w0 < tr1) {
        const int64_t nw = min((int64_t)NW, tr1 - w0);
        TSP_PUBLISH_HDR(0, w0, hdr)
        __syncthreads();
        const int ncol = sm.hs(0)[nw];
        const int64_t sbase = A.tr_slot[w0];
        TSP_ISSUE(0, sbase, ncol)
        TSP_BUILD(0, sbase, ncol)
        cp_async_wait_all();
        __syncthreads();
    }
    while (w0 < tr1) {
        const int64_t nw = min((int64_t)NW, tr1 - w0);
        const int64_t w1 = w0 + nw;
        // prefetch window k+1: header, slot bytes (cp.async), column words (registers)
        int ncol1 = 0;
        int64_t sbase1 = 0;
        if (w1 < tr1) {
            TSP_FETCH_HDR(w1, hdr)
            TSP_PUBLISH_HDR(stage ^ 1, w1, hdr)
            __syncthreads();
            const int64_t nw1 = min((int64_t)NW, tr1 - w1);
            ncol1 = sm.hs(stage ^ 1)[nw1];
            sbase1 = A.tr_slot[w1];
            TSP_ISSUE(stage ^ 1, sbase1, ncol1)
        }
        // compute window k: half-warp h owns rows w0 + h and w0 + H + h
        {
            const int32_t* hs = sm.hs(stage);
            for (int li = h; li < nw; li += H) {
                const int a = hs[li], W = hs[li + 1] - a;
                const double acc = ts_row<COUNT>(sm.ss(stage), sm.rec(stage), a, W, lane, x, cnt);
                emit(w0 + li, lane, acc);
            }
        }
        if (w1 < tr1) TSP_BUILD(stage ^ 1, sbase1, ncol1)
        cp_async_wait_all();
        __syncthreads();
        stage ^= 1;
        w0 = w1;
    }
#undef TSP_FETCH_HDR
#undef TSP_PUBLISH_HDR
#undef TSP_ISSUE
#undef TSP_BUILD
}

__device__ __forceinline__ void carve_spmv(unsigned char* base, WinSmem& w, TsSmem& ts) {
    unsigned char* p = base;
    w.misc = reinterpret_cast<int64_t*>(p);
    p += 4 * 8 + 8;
    w.pb = reinterpret_cast<unsigned long long*>(p);
    p += 4 * 8;
    w.hs = reinterpret_cast<int32_t*>(p);
    p += (WIN_TR + 1) * 4;
    w.ht = reinterpret_cast<int32_t*>(p);
    p += (WIN_TR + 1) * 4;
    p = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(p) + 15) & ~uintptr_t(15));
    w.buf = p;
    ts.base = base;
}

// emit(TR, lane, value) is called by every lane for each of its tile rows, in ascending TR.
// seg_lo/seg_hi: the column segments this CTA's tiles gather (tile-synchronous level staging).
template <bool DYN, bool COUNT, int PF, class Emit>
__device__ __forceinline__ void spmv_cta(const Mat& A, int64_t tr0, int64_t tr1, const double* x, const uint8_t* __restrict__ level,
                         int range_guard, const WinSmem& w, const TsSmem& tsm, Counts* cnt, int32_t seg_lo,
                         int32_t seg_hi, Emit emit) {
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
    // tile-synchronous slices whose windows of 2H tile rows fit the staging buffers
    if (A.ts && (int64_t)A.max_w * 2 * H <= min(TSP_COLS, TSP_CPT * B) && 2 * H <= 2 * 512) {
        spmv_ts_pipe<DYN, COUNT>(A, tr0, tr1, x, level, range_guard, tsm, cnt, seg_lo, seg_hi, emit);
        return;
    }
    uint8_t* ss = w.buf;
    uint32_t* cw = reinterpret_cast<uint32_t*>(w.buf + COL_CAP * 16);
    uint8_t* lev_s = w.buf + COL_CAP * 16 + COL_CAP * 4;
    const int32_t nlev = seg_hi - seg_lo + 1;
    const bool lev_staged = DYN && A.ts && nlev > 0 && nlev <= LEV_CAP;
    __syncthreads();
    if (t < 4) w.pb[t] = t == 0 ? (unsigned long long)A.p64 : t == 1 ? (unsigned long long)A.p32
                       : t == 2 ? (unsigned long long)A.p16 : (unsigned long long)A.p8;
    if (lev_staged)
        for (int i = t; i < nlev; i += B) lev_s[i] = level[seg_lo + i];
    for (int64_t w0 = tr0; w0 < tr1;) {
        const int64_t wmax = min(tr1 - w0, (int64_t)WIN_TR);
        __syncthreads();   // previous window fully consumed
        const int64_t s0 = A.tr_slot[w0], t0 = A.tr_tile[w0];
        for (int i = t; i <= wmax; i += B) {
            w.hs[i] = (int32_t)(A.tr_slot[w0 + i] - s0);
            w.ht[i] = (int32_t)(A.tr_tile[w0 + i] - t0);
        }
        __syncthreads();
        if (t == 0) {
            // largest multiple of H (or the whole rest) whose tiles / columns fit the buffer
            const int32_t* lim = A.ts ? w.hs : w.ht;
            const int cap = A.ts ? COL_CAP : CODE_CAP;
            int64_t nw = wmax;
            if (lim[nw] > cap) {
                nw = (int64_t)H;
                while (nw + H <= wmax && lim[nw + H] <= cap) nw += H;
                if (nw > wmax) nw = wmax;
            }
            w.misc[2] = nw;
            w.misc[3] = lim[nw] <= cap;
        }
        __syncthreads();
        const int64_t nw = w.misc[2];
        const bool staged = w.misc[3] != 0;
        const int nt = w.ht[nw];
        if (A.ts) {
            const int ncol = w.hs[nw];
            if (COUNT)
                for (int i = t; i < nt; i += B) cnt->tile(tile_code<DYN>(A.tile_info[t0 + i], level, range_guard) & 7u);
            if (staged) {
                for (int c = t; c < ncol; c += B) cp_async16(ss + c * 16, A.sslot + (s0 + c) * 16);
                for (int c = t; c < ncol; c += B)     // column words -> column codes (tc << 3 | e_t)
                    cw[c] = col_code<DYN>(__ldg(A.colw + s0 + c), lev_s, seg_lo, lev_staged, level, range_guard);
                cp_async_wait_all();
            }
            __syncthreads();
            for (int64_t li = h; li < nw; li += H) {
                const int32_t a = w.hs[li];
                const int W = w.hs[li + 1] - a;
                const int64_t sb = s0 + a;
                double acc = 0.0;
                for (int k = 0; k < W; k += PF) {
                    if (staged) {
                        acc = ts_block<COUNT, PF>(A, w.pb, ss + (a + k) * 16, cw + a + k, min(W - k, PF), lane,
                                                  (sb + k) * 16 + lane, x, acc, cnt);
                    } else {
                        uint32_t cdl[PF];
#pragma unroll
                        for (int q = 0; q < PF; ++q)
                            cdl[q] = k + q < W ? col_code<DYN>(__ldg(A.colw + sb + k + q), lev_s, seg_lo, lev_staged, level,
                                                                range_guard) : (uint32_t)BYP;
                        acc = ts_block<COUNT, PF>(A, w.pb, A.sslot + (sb + k) * 16, cdl, min(W - k, PF), lane,
                                                  (sb + k) * 16 + lane, x, acc, cnt);
                    }
                }
                emit(w0 + li, lane, acc);
            }
            w0 += nw;
            continue;
        }
        uint32_t* code = reinterpret_cast<uint32_t*>(w.buf);
        for (int i = t; i < nt; i += B) {
            const uint32_t c = tile_code<DYN>(A.tile_info[t0 + i], level, range_guard);
            if (staged) code[i] = c;
            if (COUNT) cnt->tile((int)(c & 7u));
        }
        __syncthreads();
        // half-warp h: tile rows w0 + h + kH, the next row's first PF slot words prefetched
        uint16_t nxt[PF];
        int64_t li = h;
#define CMP_LOAD_FIRST(L)                                                                           {                                                                                               const int32_t a_ = w.hs[L], W_ = w.hs[(L) + 1] - a_;                                        const uint16_t* sp_ = A.sidx + (s0 + a_) * 16 + lane;                                       _Pragma("unroll") for (int q = 0; q < PF; ++q) nxt[q] = q < W_ ? __ldg(sp_ + q * 16) : mf::SLOT_PAD;         }
        if (li < nw) CMP_LOAD_FIRST(li)
        for (; li < nw; li += H) {
            uint16_t cur[PF];
#pragma unroll
            for (int q = 0; q < PF; ++q) cur[q] = nxt[q];
            if (li + H < nw) CMP_LOAD_FIRST(li + H)
            const int32_t a = w.hs[li];
            const int W = w.hs[li + 1] - a;
            const int64_t sb = s0 + a;
            const int64_t tb_abs = t0 + w.ht[li];
            const uint32_t* cd = code + w.ht[li];
            double acc = 0.0;
            acc = slot_block<DYN, COUNT, PF>(A, w.pb, cur, min(W, PF), sb * 16 + lane, cd, staged, tb_abs, level,
                                              range_guard, x, acc, cnt);
            for (int k = PF; k < W; k += PF) {
                uint16_t more[PF];
                const uint16_t* sp = A.sidx + (sb + k) * 16 + lane;
#pragma unroll
                for (int q = 0; q < PF; ++q) more[q] = (k + q < W) ? __ldg(sp + q * 16) : mf::SLOT_PAD;
                acc = slot_block<DYN, COUNT, PF>(A, w.pb, more, min(W - k, PF), (sb + k) * 16 + lane, cd, staged, tb_abs,
                                                  level, range_guard, x, acc, cnt);
            }
            emit(w0 + li, lane, acc);
        }
#undef CMP_LOAD_FIRST
        w0 += nw;
    }
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
