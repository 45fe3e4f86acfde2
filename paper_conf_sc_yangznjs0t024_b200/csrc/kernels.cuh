// kernels.cuh -- device building blocks shared by the persistent solver kernels and the
// standalone mf_spmv / mf_levels / mf_dot kernels.
//
//  * spmv_ts / spmv_compact: Alg. 5.  A half-warp owns a tile row, lane r = row
//    16*TR+r; each row is ONE fma chain over its nonzeros in ascending column order (the slice
//    layouts store them in that order), so no floating-point atomics are needed (Alg. 5 l.13's
//    atomicAdd disappears) and the result is bit-identical for any launch shape.
//  * level_of / tile_code: Alg. 4 thresholds and the effective precision e_t.
//  * Reductions: the fixed tree of DESIGN.md "Reduction order" (thread fma chain -> warp
//    xor-butterfly -> tree32 over warps -> tree32 over CTAs).
#pragma once

#include "mf_internal.cuh"

namespace mfk {

constexpr int BYP = 4;

struct TsStage;

struct Mat {
    int64_t n_rows, n_cols, ntr;
    const int64_t* __restrict__ tr_slot;
    const int64_t* __restrict__ tr_tile;
    const uint32_t* __restrict__ tile_info;
    const uint16_t* __restrict__ sidx;    // compact layout
    const uint8_t* __restrict__ blob;     // tile-synchronous layout: per-stage blobs (the TMA source)
    const TsStage* __restrict__ stg;      // stages of every CTA
    const int32_t* __restrict__ stg_ptr;  // [G+1]
    const int64_t* __restrict__ tile_nnz; // TileNnz (canonical)
    int ts;
    int max_w;                            // widest tile-row slice (slice columns)
    const double* __restrict__ p64;
    const float* __restrict__ p32;
    const __half* __restrict__ p16;
    const uint8_t* __restrict__ p8;
    uint8_t* stk;                         // sticky variant (P:237 literal): per slice column (TS layout) or
                                          // per tile (compact), bit L set = values lowered to L in place
    int64_t coff;                         // column segment of row segment 0 (row-block ranks: the halo
                                          // segments of lower ranks precede the own ones); 0 = square
};

// ------------------------------------------------------------------------------------------
// SpMV input vectors ("PV" layout).  Every vector that feeds an SpMV inside the solver (p, s,
// p^, s^) is stored as 16-element segments of 144 bytes: 16 binary64 values, then the segment's
// level byte (Alg. 4: 0 FP64 .. 3 FP8, 4 bypass) in the low byte of element 16,
// element 17 padding.  The producer of the vector (the CTA that owns the rows) writes the
// level next to the values, so one bulk copy of a run of segments stages both the x values and
// the tile-column levels of an SpMV stage (the "vis_flag" of Alg. 5 l.2) in shared memory.
constexpr int PVS = 18;                      // doubles per segment
constexpr int PV_SEG_BYTES = PVS * 8;        // 144
__host__ __device__ __forceinline__ int64_t pv_idx(int64_t i) { return (i >> 4) * PVS + (i & 15); }
__device__ __forceinline__ int pv_level(const double* pv, int64_t seg) {
    return (int)reinterpret_cast<const uint8_t*>(pv + seg * PVS + 16)[0];
}
__device__ __forceinline__ void pv_set_level(double* pv, int64_t seg, int lv) {
    reinterpret_cast<uint8_t*>(pv + seg * PVS + 16)[0] = (uint8_t)lv;
}

__device__ __forceinline__ unsigned hw_mask() { return (threadIdx.x & 16) ? 0xFFFF0000u : 0x0000FFFFu; }

// min over the half-warp (mask m): one redux.sync
__device__ __forceinline__ int hw_min_i(int v, unsigned m) { return (int)__reduce_min_sync(m, (unsigned)v); }
// the same for a level (0..4) when all 32 lanes are present: two full-warp reductions, each half
// feeding the neutral 4 into the other's (no per-half masks, no divergence checks)
__device__ __forceinline__ int hw_min_level_full(int v) {
    const bool upper = (threadIdx.x & 16) != 0;
    const unsigned lo = __reduce_min_sync(0xffffffffu, upper ? 4u : (unsigned)v);
    const unsigned hi = __reduce_min_sync(0xffffffffu, upper ? (unsigned)v : 4u);
    return (int)(upper ? hi : lo);
}

// (tile column << 3) | e_t.   e_t = bypass | max_prec(floor, min_prec(TilePrec, level))
template <bool DYN>
__device__ __forceinline__ uint32_t tile_code(uint32_t info, const double* pv, int range_guard) {
    const uint32_t tc = info >> 4;
    int e = (int)(info & 3u);
    if (DYN) {
        const int lv = pv_level(pv, tc);
        if (lv == BYP) return (tc << 3) | BYP;
        e = max(e, lv);
        if (range_guard) e = min(e, (int)((info >> 2) & 3u));
    }
    return (tc << 3) | (uint32_t)e;
}

// sticky variant, compact layout (P:237 literal; oracle spmv_tiles): per-tile mask of the levels
// the tile was lowered to in place.  Code = (tile column << 3) | e_t | TilePrec << 27 | mask << 29
// (mask bits L = 1..3 stored as mask >> 1; tile column < 2^24); `update` (the window's code staging, one thread per tile) records a new
// lowering, the per-slot recomputation of an unstaged window only reads the updated mask.
__device__ __forceinline__ uint32_t sticky_code(const Mat& A, int64_t tile, const double* pv, int range_guard,
                                                bool update) {
    const uint32_t info = A.tile_info[tile];
    const uint32_t tc = info >> 4, prec = info & 3u;
    const int lv = pv_level(pv, tc);
    if (lv == BYP) return (tc << 3) | BYP;
    unsigned mask = A.stk[tile];
    const int cur = mask ? 31 - __clz(mask) : (int)prec;
    int e = max(lv, cur);
    if (range_guard) e = min(e, (int)((info >> 2) & 3u));
    if (e > cur) {
        mask |= 1u << e;
        if (update) A.stk[tile] = (uint8_t)mask;
    }
    return (tc << 3) | (uint32_t)e | (prec << 27) | ((mask >> 1) << 29);   // mask bits 1..3
}
constexpr uint32_t CODE_TC_MASK = 0x00FFFFFFu;   // tile column field of a code (after >> 3)

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
    __device__ __forceinline__ void nzn(int e, int k) {
        if (e < 3) n_lo += (unsigned long long)k << (21 * e); else n_hi += (unsigned long long)k << (21 * (e - 3));
    }
    __device__ __forceinline__ static int field(unsigned long long lo, unsigned long long hi, int q) {
        return (int)(((q < 3 ? lo : hi) >> (21 * (q < 3 ? q : q - 3))) & 0x1FFFFFull);
    }
    __device__ __forceinline__ int tiles(int q) const { return field(t_lo, t_hi, q); }
    __device__ __forceinline__ int nnz(int q) const { return field(n_lo, n_hi, q); }
};

// ------------------------------------------------------------------------------------------
// Tile-synchronous (TS) slices streamed through shared memory by the Tensor Memory Accelerator
// (cp.async.bulk + mbarrier): the B200 form of "load the tiles on chip" and of the
// on-chip precision conversion.
//
// TS layout (convert.cu): tile row TR owns slice columns; a slice column belongs to ONE tile and
// holds, for lane r = row 16*TR + r, the local column (0 on padding) and the value stored at
// TilePrec (0 on padding).  The persistent CTA owns the contiguous tile rows [tr0, tr1); half-warp
// h takes the tile rows TR = tr0 + h (mod H) (lane r = row 16*TR + r: the row mapping of the
// dot-product contract), so warp w owns the rows of half-warps 2w and 2w+1.  Conversion cuts the
// CTA's tile rows into stages (one tile row per half-warp by default) and packs each stage into
// ONE contiguous blob:
//   [int32 hdr[16]: tr0, tr1, nc, off_desc, -, off_val, own_w, col0 lo, col0 hi, off_wl, off_gd]
//   [int16 column start per tile-row boundary, K+1 entries]
//   [u32 desc per column: x offset | slot << 16; TS_DPAD padding entries]
//   [per warp uint4: column counts per TilePrec group (4 x u8), value offset, gd offset]
//   [u32 gd per column in each warp's grouped order: window byte offset | Floor << 16 | column << 20]
//   [values: per warp, its columns grouped by TilePrec (FP64 | FP32 | FP16 | E4M3), 16 x size each]
// A slice column holds ONE diagonal of its tile (local column - local row = d, diagonals in
// ascending order), so lane r's x is window element 16 w + r + d: the descriptor carries the byte
// offset of element 16 w + d from the slot's zero guard (padding lanes read finite values).  The
// decode-buffer slot of a column is its rank in the warp's grouped order, so the decode is a
// linear stream per group (no per-value indirection).
// The stage record (TsStage, 32 words) lists the runs of consecutive column segments the stage
// gathers ("x windows"); the runs are bulk-copied from the PV vector next to the blob.
//
// Per stage, every warp independently (no CTA barrier): wait the slot's "full" mbarrier; decode
// its columns group by group (warp-uniform precision, 4 values per lane, exact upcast) into its
// private FP64 buffer E_w, applying the dynamic switch of Alg. 5 (bypass -> 0; e_t below TilePrec
// -> RNE_{e_t} of the stored value: P:237's on-chip conversion); __syncwarp; each half-warp runs
// its row's single fma chain in ascending column order with E_w and x from the staged window;
// arrive on the slot's "empty" mbarrier.  Warp 0 refills a slot (one lane per bulk copy) once
// every warp has arrived.
constexpr int TS_KCAP = 64;       // tile rows per stage
constexpr int TS_CCAP = 512;      // slice columns per stage
constexpr int TS_VCAP = 16384;    // value bytes per stage
constexpr int TS_WCAP = 224;      // window segments per stage
constexpr int TS_RUNCAP = 8;      // runs per stage
constexpr int TS_NSTMAX = 6;      // slots in the ring
constexpr int TS_HDR = 64;        // blob header bytes
constexpr int TS_PF = 4;          // stage records prefetched ahead by the issuing warp
constexpr int TS_EBYTES = 98304;  // most shared memory the warp-private decode buffers may take
constexpr int TS_DPAD = 16;       // padding column descriptors after the last column (short-row reads)
constexpr int TS_GUARD = 128;     // zero bytes before each slot's x window (reads of padding lanes)
__host__ __device__ constexpr int ts_r16(int v) { return (v + 15) & ~15; }

// stage record: 32 words, word l read by lane l of the issuing warp
struct TsStage {
    uint32_t boff_lo, boff_hi;      // blob offset in Mat::blob
    int32_t bbytes;                 // blob bytes (multiple of 16)
    int32_t nrun, wseg;             // runs, window segments (sum of run lengths)
    int32_t tr0, tr1, nc;
    int32_t run_s[TS_RUNCAP];       // first segment of each run
    int32_t run_n[TS_RUNCAP];       // segments of each run
    int32_t run_w[TS_RUNCAP];       // window offset (segments) of each run
};
static_assert(sizeof(TsStage) == 128, "TsStage is 32 words");

struct TsSmem {
    unsigned char* base;            // ring of nst slots of slot_bytes
    double* ebuf;                   // per-warp decode buffers: ecap columns x 16 doubles per warp
    int nst, slot_bytes, blob_cap, ecap;
    unsigned long long* full;       // [TS_NSTMAX]
    unsigned long long* empty;      // [TS_NSTMAX] release counters: warps done with the slot's stage
    unsigned long long* ctr;        // [0] stages issued so far (ring position); [1] resident SpMVs done
    __device__ __forceinline__ unsigned char* slot(int s) const { return base + (size_t)s * slot_bytes; }
};
constexpr size_t TS_CTRL_BYTES = 16 * TS_NSTMAX + 32;

__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, unsigned cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ bool mbar_try(unsigned long long* b, unsigned parity) {
    unsigned ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(b)), "r"(parity) : "memory");
    return ok != 0;
}
// bounded wait: a pipeline that cannot complete traps (kernel error) instead of hanging the GPU
__device__ __forceinline__ bool mbar_try_suspend(unsigned long long* b, unsigned parity) {
    unsigned ok;
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(b)), "r"(parity), "r"(2000u) : "memory");
    return ok != 0;
}
static __device__ __noinline__ void mbar_wait_slow(unsigned long long* b, unsigned parity) {
    unsigned long long t0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    for (unsigned k = 1;; ++k) {
        // try_wait suspends the warp in hardware until the phase completes or a time limit passes:
        // the loop issues a few instructions per wake-up, the timer is read rarely
        if (mbar_try(b, parity)) return;
        if ((k & 1023u) == 0) {
            unsigned long long t1;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
            if (t1 - t0 > 20ull * 1000000000ull) __trap();
        }
    }
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, unsigned parity) {
    if (!mbar_try(b, parity)) mbar_wait_slow(b, parity);
}
__device__ __forceinline__ unsigned long long policy_evict_first() {
    unsigned long long p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// the matrix is read once per SpMV -> L2 evict_first (keeps the solver's vectors L2-resident)
__device__ __forceinline__ void bulk_g2s_ef(void* dst, const void* src, unsigned bytes, unsigned long long* bar,
                                            unsigned long long pol) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, unsigned long long* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

// all threads; followed by a __syncthreads of the caller before the first SpMV
__device__ __forceinline__ void ts_init(const TsSmem& sm) {
    for (int s = 0; s < sm.nst; ++s)      // the zero guard before each slot's window (never a TMA target)
        for (int i = threadIdx.x; i < TS_GUARD / 8; i += blockDim.x)
            reinterpret_cast<double*>(sm.slot(s) + sm.blob_cap)[i] = 0.0;
    if (threadIdx.x == 0) {
        for (int s = 0; s < TS_NSTMAX; ++s) {
            mbar_init(sm.full + s, 1);
            sm.empty[s] = 0ull;       // release counter of the slot (warps done with it)
        }
        sm.ctr[0] = 0ull;
        sm.ctr[1] = 0ull;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
}

// Warp 0: stage record word l in lane l (rec).  Lane 0 posts the transaction bytes, then lane r
// (r < nrun) copies window run r and lane 31 the blob.
__device__ __forceinline__ void ts_issue(const unsigned char* blob_base, uint32_t rec, unsigned char* slot, int blob_cap,
                                         unsigned long long* full, const double* pv, bool with_blob, unsigned long long pol) {
    const int lane = threadIdx.x & 31;
    const uint32_t boff_lo = __shfl_sync(0xffffffffu, rec, 0), boff_hi = __shfl_sync(0xffffffffu, rec, 1);
    const int bbytes = (int)__shfl_sync(0xffffffffu, rec, 2), nrun = (int)__shfl_sync(0xffffffffu, rec, 3);
    const int wseg = (int)__shfl_sync(0xffffffffu, rec, 4);
    const int rs = (int)__shfl_sync(0xffffffffu, rec, 8 + (lane & 7));
    const int rn = (int)__shfl_sync(0xffffffffu, rec, 16 + (lane & 7));
    const int rw = (int)__shfl_sync(0xffffffffu, rec, 24 + (lane & 7));
    if (lane == 0) mbar_expect_tx(full, (unsigned)((with_blob ? bbytes : 0) + wseg * PV_SEG_BYTES));
    __syncwarp();
    if (lane < nrun && lane < TS_RUNCAP)
        bulk_g2s(slot + blob_cap + TS_GUARD + rw * PV_SEG_BYTES, pv + (int64_t)rs * PVS, (unsigned)(rn * PV_SEG_BYTES), full);
    if (lane == 31 && with_blob) {
        const uint64_t boff = ((uint64_t)boff_hi << 32) | boff_lo;
        bulk_g2s_ef(slot, blob_base + boff, (unsigned)bbytes, full, pol);
    }
}

// exact upcast of the stored bits at precision e (0 FP64, 1 FP32, 2 FP16, 3 E4M3) to binary64
__device__ __forceinline__ double f16b_to_f64(unsigned short b);
__device__ __forceinline__ uint32_t e4m3x2_to_f16x2(uint32_t w);
__device__ __forceinline__ double decode_val(int e, uint64_t raw) {
    const uint32_t lo = (uint32_t)raw;
    const unsigned short hb = e == 3 ? (unsigned short)e4m3x2_to_f16x2(lo & 0xFFu) : (unsigned short)lo;
    const double d = e >= 2 ? f16b_to_f64(hb) : (double)__uint_as_float(lo);
    return e == 0 ? __longlong_as_double((long long)raw) : d;
}
// binary16 bits -> binary64 (exact; one F2F.F64.F16)
__device__ __forceinline__ double f16b_to_f64(unsigned short b) {
    double d;
    asm("{\n\t.reg .f16 h;\n\tmov.b16 h, %1;\n\tcvt.f64.f16 %0, h;\n\t}" : "=d"(d) : "h"(b));
    return d;
}
// two E4M3 bytes (bits 0..15 of w) -> two binary16 (exact; one F2FP.F16.E4M3.UNPACK_B), byte 0 in the low half
__device__ __forceinline__ uint32_t e4m3x2_to_f16x2(uint32_t w) {
    uint32_t r;
    asm("cvt.rn.f16x2.e4m3x2 %0, %1;" : "=r"(r) : "h"((unsigned short)(w & 0xFFFFu)));
    return r;
}
__device__ __forceinline__ double e4m3_lo(uint32_t w2) {   // the E4M3 byte in bits 0..7 -> binary64 (exact)
    const __half_raw h = __nv_cvt_fp8_to_halfraw((__nv_fp8_storage_t)(w2 & 0xFFu), __NV_E4M3);
    return (double)__half2float(__half(h));
}
__device__ __forceinline__ double h16(uint32_t bits) { return (double)__half2float(__ushort_as_half((unsigned short)bits)); }
__device__ __forceinline__ float f16f(uint32_t bits) { return __half2float(__ushort_as_half((unsigned short)bits)); }
__device__ __forceinline__ float e4m3f(uint32_t w2) {      // the E4M3 byte in bits 0..7 -> binary32 (exact)
    const __half_raw h = __nv_cvt_fp8_to_halfraw((__nv_fp8_storage_t)(w2 & 0xFFu), __NV_E4M3);
    return __half2float(__half(h));
}

// view of one landed stage (header: three 16-byte loads)
struct TsView {
    const unsigned char* blob;
    const double* win;
    int S0, S1, off_desc, off_val, own_w, off_wl, off_gd, off0;
    int64_t col0;
};
__device__ __forceinline__ TsView ts_view(const unsigned char* slot, int blob_cap) {
    TsView v;
    const int4 h0 = reinterpret_cast<const int4*>(slot)[0];
    const int4 h1 = reinterpret_cast<const int4*>(slot)[1];
    const int4 h2 = reinterpret_cast<const int4*>(slot)[2];
    v.blob = slot;
    v.win = reinterpret_cast<const double*>(slot + blob_cap + TS_GUARD);
    v.S0 = h0.x; v.S1 = h0.y; v.off_desc = h0.w;
    v.off_val = h1.y; v.own_w = h1.z;
    v.col0 = (int64_t)(((uint64_t)(uint32_t)h2.x << 32) | (uint32_t)h1.w);
    v.off_wl = h2.y; v.off_gd = h2.z; v.off0 = h2.w;
    return v;
}

// the dynamic switch for 4 decoded values whose segment level lv exceeds their TilePrec q:
// bypass -> 0; else RNE at e_t = min(lv, floor) when that is below q (range guard R19)
struct D4 {
    double a, b, c, d;
};
static __device__ __noinline__ D4 ts_lower4(D4 w, int lv, int floor_, int q) {
    if (lv == BYP) return D4{0.0, 0.0, 0.0, 0.0};
    const int e = min(lv, floor_);
    if (e == q) return w;
    return D4{round_to(w.a, e), round_to(w.b, e), round_to(w.c, e), round_to(w.d, e)};
}

// Decode of one warp's group of n columns at TilePrec Q (warp-uniform) into its buffer E: values
// vb[0 .. 16n) -> E[slot0*16 ..), 4 values per lane per step, exact upcast.  Dynamic switch (Alg. 5
// l.2-4, range guard R19): bypass -> 0, e_t below TilePrec -> RNE_{e_t}(stored).  Sticky variant
// (P:237 literal): the column's mask of the levels it was lowered to in place (Mat::stk, per slice
// column); the working value is RNE applied at every lowered level in ascending order.
template <int Q, bool DYN, bool STK>
__device__ __forceinline__ void ts_decode_group(const TsView& v, const unsigned char* vb, const uint32_t* gd, int n, double* E,
                                                int range_guard, uint8_t* stk) {
    const int lane = threadIdx.x & 31;
    for (int u = lane; u < 4 * n; u += 32) {
        const unsigned char* src = vb + (u << (5 - Q));
        double w[4];
        if (Q == 0) {
            const double2 a = reinterpret_cast<const double2*>(src)[0], b = reinterpret_cast<const double2*>(src)[1];
            w[0] = a.x; w[1] = a.y; w[2] = b.x; w[3] = b.y;
        } else if (Q == 1) {
            const float4 a = *reinterpret_cast<const float4*>(src);
            w[0] = (double)a.x; w[1] = (double)a.y; w[2] = (double)a.z; w[3] = (double)a.w;
        } else if (Q == 2) {
            const uint2 a = *reinterpret_cast<const uint2*>(src);
            w[0] = f16b_to_f64((unsigned short)a.x); w[1] = f16b_to_f64((unsigned short)(a.x >> 16));
            w[2] = f16b_to_f64((unsigned short)a.y); w[3] = f16b_to_f64((unsigned short)(a.y >> 16));
        } else {
            const uint32_t a = *reinterpret_cast<const uint32_t*>(src);
            const uint32_t h01 = e4m3x2_to_f16x2(a), h23 = e4m3x2_to_f16x2(a >> 16);
            w[0] = f16b_to_f64((unsigned short)h01); w[1] = f16b_to_f64((unsigned short)(h01 >> 16));
            w[2] = f16b_to_f64((unsigned short)h23); w[3] = f16b_to_f64((unsigned short)(h23 >> 16));
        }
        if (DYN) {
            const uint32_t g = gd[u >> 2];
            const int lv = (int)(reinterpret_cast<const uint8_t*>(v.win) + (g & 0xFFFFu))[128];
            if (STK) {
                if (lv == BYP) { w[0] = w[1] = w[2] = w[3] = 0.0; }
                else {
                    uint8_t* sp = stk + (v.col0 + (int)(g >> 20));
                    unsigned mask = *sp;
                    const int cur = mask ? 31 - __clz(mask) : Q;
                    int e = max(lv, cur);
                    if (range_guard) e = min(e, (int)((g >> 16) & 3u));
                    if (e > cur) {
                        mask |= 1u << e;
                        if ((u & 3) == 0) *sp = (uint8_t)mask;   // every unit of the column computes the same mask
                    }
#pragma unroll
                    for (int L = Q + 1; L <= 3; ++L)
                        if (mask & (1u << L)) {
#pragma unroll
                            for (int k = 0; k < 4; ++k) w[k] = round_to(w[k], L);
                        }
                }
            } else if (lv > Q) {
                // rare path out of line: keeps the hot decode loop small (instruction cache)
                const D4 r = ts_lower4(D4{w[0], w[1], w[2], w[3]}, lv, range_guard ? (int)((g >> 16) & 3u) : 3, Q);
                w[0] = r.a; w[1] = r.b; w[2] = r.c; w[3] = r.d;
            }
        }
        // the two 16-byte halves in a lane-rotated order: conflict-free shared stores
        double2* ea = reinterpret_cast<double2*>(E + u * 4);
        if ((u >> 2) & 1) {
            ea[1] = make_double2(w[2], w[3]);
            ea[0] = make_double2(w[0], w[1]);
        } else {
            ea[0] = make_double2(w[0], w[1]);
            ea[1] = make_double2(w[2], w[3]);
        }
    }
}

// One tile row of this half-warp, N = the warp's widest row: columns beyond W read the next
// descriptors (or the padding ones) and contribute fma(0, x, acc) == acc exactly (acc is never -0,
// x is finite), so both half-warps run the same instruction stream.  Per column: the descriptor
// (LDS, immediate offset), x of the lane's diagonal from the window, the decoded value from the
// warp's buffer, one fma in ascending column order.
struct TsRowCtx {
    const uint32_t* desc;
    const unsigned char* xw;        // slot's window guard + lane * 8
    const double* el;               // warp's decode buffer + lane
};
template <int N>
__device__ __forceinline__ double ts_row(const TsRowCtx& r, int a, int W) {
    double ev[N], xv[N];
#pragma unroll
    for (int q = 0; q < N; ++q) {
        const uint32_t d = r.desc[a + q];
        ev[q] = q < W ? r.el[(d >> 16) * 16] : 0.0;
        xv[q] = *reinterpret_cast<const double*>(r.xw + (d & 0xFFFFu));
    }
    double acc = 0.0;
#pragma unroll
    for (int q = 0; q < N; ++q) acc = __fma_rn(ev[q], xv[q], acc);
    return acc;
}
__device__ __forceinline__ double ts_row_long(const TsRowCtx& r, int a, int W) {
    double acc = 0.0;
    for (int q = 0; q < W; ++q) {
        const uint32_t d = r.desc[a + q];
        acc = __fma_rn(r.el[(d >> 16) * 16], *reinterpret_cast<const double*>(r.xw + (d & 0xFFFFu)), acc);
    }
    return acc;
}
__device__ __forceinline__ double ts_row_any(const TsRowCtx& r, int a, int W, int Wmax) {
    switch (Wmax) {
    case 0: return 0.0;
    case 1: return ts_row<1>(r, a, W);
    case 2: return ts_row<2>(r, a, W);
    case 3: return ts_row<3>(r, a, W);
    case 4: return ts_row<4>(r, a, W);
    case 5: return ts_row<5>(r, a, W);
    case 6: return ts_row<6>(r, a, W);
    case 7: return ts_row<7>(r, a, W);
    case 8: return ts_row<8>(r, a, W);
    case 9: return ts_row<9>(r, a, W);
    case 10: return ts_row<10>(r, a, W);
    case 11: return ts_row<11>(r, a, W);
    case 12: return ts_row<12>(r, a, W);
    default: return ts_row_long(r, a, W);
    }
}
// two tile rows of this half-warp at once (independent fma chains: ILP 2)
template <int N>
__device__ __forceinline__ void ts_row2(const TsRowCtx& r, int a1, int W1, int a2, int W2, double& acc1, double& acc2) {
    double e1[N], x1[N], e2[N], x2[N];
#pragma unroll
    for (int q = 0; q < N; ++q) {
        const uint32_t d1 = r.desc[a1 + q], d2 = r.desc[a2 + q];
        e1[q] = q < W1 ? r.el[(d1 >> 16) * 16] : 0.0;
        e2[q] = q < W2 ? r.el[(d2 >> 16) * 16] : 0.0;
        x1[q] = *reinterpret_cast<const double*>(r.xw + (d1 & 0xFFFFu));
        x2[q] = *reinterpret_cast<const double*>(r.xw + (d2 & 0xFFFFu));
    }
    double s1 = 0.0, s2 = 0.0;
#pragma unroll
    for (int q = 0; q < N; ++q) {
        s1 = __fma_rn(e1[q], x1[q], s1);
        s2 = __fma_rn(e2[q], x2[q], s2);
    }
    acc1 = s1;
    acc2 = s2;
}
__device__ __forceinline__ void ts_row2_any(const TsRowCtx& r, int a1, int W1, int a2, int W2, int Wmax, double& acc1, double& acc2) {
    switch (Wmax) {
    case 0: acc1 = acc2 = 0.0; return;
    case 1: ts_row2<1>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 2: ts_row2<2>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 3: ts_row2<3>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 4: ts_row2<4>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 5: ts_row2<5>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 6: ts_row2<6>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 7: ts_row2<7>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 8: ts_row2<8>(r, a1, W1, a2, W2, acc1, acc2); return;
    case 9: ts_row2<9>(r, a1, W1, a2, W2, acc1, acc2); return;
    default:
        acc1 = ts_row_long(r, a1, W1);
        acc2 = ts_row_long(r, a2, W2);
        return;
    }
}

// consume one landed stage (one warp): decode its columns, then the rows of its two half-warps.
// own_mode: 0 none; 1 the SpMV input at the row (from the window when the stage's own segments
// are staged); 2 the normal vector `ownv`.
template <bool DYN, bool STK, class Emit>
__device__ __forceinline__ void ts_consume(const TsView& v, const double* pv, int range_guard, int own_mode, const double* ownv,
                                           int64_t n, uint8_t* stk, double* E, Emit& emit) {
    const int t = threadIdx.x, H = blockDim.x >> 4, h = t >> 4, lane = t & 15, w = t >> 5;
    {
        const uint4 wl = reinterpret_cast<const uint4*>(v.blob + v.off_wl)[w];
        const int n0 = wl.x & 0xFF, n1 = (wl.x >> 8) & 0xFF, n2 = (wl.x >> 16) & 0xFF, n3 = wl.x >> 24;
        const unsigned char* vb = v.blob + v.off_val + wl.y;
        const uint32_t* gd = reinterpret_cast<const uint32_t*>(v.blob + v.off_gd) + wl.z;
        ts_decode_group<0, DYN, STK>(v, vb, gd, n0, E, range_guard, stk);
        vb += n0 * 128; gd += n0;
        ts_decode_group<1, DYN, STK>(v, vb, gd, n1, E + n0 * 16, range_guard, stk);
        vb += n1 * 64; gd += n1;
        ts_decode_group<2, DYN, STK>(v, vb, gd, n2, E + (n0 + n1) * 16, range_guard, stk);
        vb += n2 * 32; gd += n2;
        ts_decode_group<3, DYN, STK>(v, vb, gd, n3, E + (n0 + n1 + n2) * 16, range_guard, stk);
    }
    __syncwarp();
    const int16_t* cs = reinterpret_cast<const int16_t*>(v.blob + TS_HDR);
    TsRowCtx rc;
    rc.desc = reinterpret_cast<const uint32_t*>(v.blob + v.off_desc);
    rc.xw = reinterpret_cast<const unsigned char*>(v.win) - TS_GUARD + lane * 8;
    rc.el = E + lane;
    auto emit_row = [&](int k, double acc) {
        const int TR = v.S0 + k;
        double ov = 0.0;
        if (own_mode == 1) ov = v.own_w >= 0 ? v.win[(v.own_w + k) * PVS + lane] : pv[(int64_t)TR * PVS + lane];
        else if (own_mode == 2) {
            const int64_t i = (int64_t)TR * 16 + lane;
            if (i < n) ov = ownv[i];
        }
        emit((int64_t)TR, lane, acc, ov);
    };
    // rows k and k + H of this half-warp together (two chains); both half-warps of the warp run the
    // same iterations (their rows or nothing).  off0 = (S0 - tr0c) mod H (conversion).
    const int nrow = v.S1 - v.S0;
    for (int k = h >= v.off0 ? h - v.off0 : h - v.off0 + H;; k += 2 * H) {
        const bool m1 = k < nrow, m2 = k + H < nrow;
        if (!__any_sync(0xffffffffu, m1)) break;
        const int a1 = m1 ? cs[k] : 0, W1 = m1 ? cs[k + 1] - a1 : 0;
        const int a2 = m2 ? cs[k + H] : 0, W2 = m2 ? cs[k + H + 1] - a2 : 0;
        int Wm = max(W1, W2);
        Wm = max(Wm, __shfl_xor_sync(0xffffffffu, Wm, 16));
        if (__any_sync(0xffffffffu, m2)) {
            double acc1, acc2;
            ts_row2_any(rc, a1, W1, a2, W2, Wm, acc1, acc2);
            if (m1) emit_row(k, acc1);
            if (m2) emit_row(k + H, acc2);
        } else {
            const double acc1 = ts_row_any(rc, a1, W1, Wm);
            if (m1) emit_row(k, acc1);
        }
    }
    __syncwarp();
}

// The whole SpMV of one CTA (all threads), tile rows [tr0c, tr1c) = the CTA's plan range, input
// vector pv (PV layout, levels included).  Called with every thread of the CTA; the caller
// guarantees pv is complete (ready flags / barrier).
template <bool DYN, bool STK, class Emit>
__device__ __forceinline__ void spmv_ts(const Mat& A, int64_t tr0c, const double* pv, int range_guard, const TsSmem& sm,
                                        int own_mode, const double* ownv, Emit& emit) {
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    const int32_t s_begin = A.stg_ptr[blockIdx.x], ns = A.stg_ptr[blockIdx.x + 1] - s_begin;
    const uint32_t* recs = reinterpret_cast<const uint32_t*>(A.stg + s_begin);
    const int NST = sm.nst;
    double* E = sm.ebuf + (size_t)w * sm.ecap * 16;     // decode buffer: ecap columns x 16 doubles
    const double* xb = pv - A.coff * PVS;                 // column space (pv: the own segments)
    __syncthreads();                          // ring counters / previous phase's smem users
    if (ns == 0) return;
    unsigned long long pol = 0;
    if (w == 0) {
        pol = policy_evict_first();
        asm volatile("fence.proxy.async.global;" ::: "memory");   // generic-proxy writes of pv -> bulk copies
    }
    if (ns <= NST) {
        // every stage of this CTA fits the ring: the blobs stay resident across SpMVs (small
        // matrices, e.g. C1); only the x windows are re-staged
        const unsigned rc = (unsigned)sm.ctr[1];
        if (w == 0)
            for (int k = 0; k < ns; ++k) ts_issue(A.blob, recs[k * 32 + lane], sm.slot(k), sm.blob_cap, sm.full + k, xb, rc == 0, pol);
        for (int k = 0; k < ns; ++k) {
            mbar_wait(sm.full + k, rc & 1u);
            ts_consume<DYN, STK>(ts_view(sm.slot(k), sm.blob_cap), pv, range_guard, own_mode, ownv, A.n_rows, A.stk, E, emit);
        }
        __syncthreads();
        if (t == 0) sm.ctr[1] = rc + 1;
        return;
    }
    // streaming: ring position u0 (slot = u mod NST, phase = (u / NST) & 1), 32-bit counters.
    // Warp 0 fills the ring; afterwards the LAST warp to release a slot (a shared-memory counter per
    // slot) refills it with stage k + NST, so no warp ever waits for the others to drain a slot.
    // Every warp reads the record of stage k + NST while it waits for stage k (one word per lane).
    const unsigned u0 = (unsigned)sm.ctr[0];
    const unsigned NW = blockDim.x >> 5;
    int sl = (int)(u0 % (unsigned)NST);
    unsigned ph = (u0 / (unsigned)NST) & 1u;
    if (w == 0) {
        int isl = sl;
        for (int k = 0; k < min(ns, NST); ++k) {
            ts_issue(A.blob, recs[k * 32 + lane], sm.slot(isl), sm.blob_cap, sm.full + isl, xb, true, pol);
            if (++isl == NST) isl = 0;
        }
    }
    for (int k = 0; k < ns; ++k) {
        const bool refill = k + NST < ns;
        const uint32_t rnext = refill ? __ldg(recs + (size_t)(k + NST) * 32 + lane) : 0u;
        mbar_wait(sm.full + sl, ph);
        ts_consume<DYN, STK>(ts_view(sm.slot(sl), sm.blob_cap), pv, range_guard, own_mode, ownv, A.n_rows, A.stk, E, emit);
        unsigned old = 0;
        if (lane == 0) {
            __threadfence_block();                                   // release: this warp's reads of the slot
            old = atomicAdd(reinterpret_cast<unsigned*>(sm.empty + sl), 1u);
        }
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old == NW - 1) {                                         // every warp is done with the slot
            if (lane == 0) {
                *reinterpret_cast<volatile unsigned*>(sm.empty + sl) = 0u;
                __threadfence_block();                               // acquire: the other warps' reads
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            }
            __syncwarp();
            if (refill) {
                if (pol == 0) {
                    pol = policy_evict_first();
                    asm volatile("fence.proxy.async.global;" ::: "memory");
                }
                ts_issue(A.blob, rnext, sm.slot(sl), sm.blob_cap, sm.full + sl, xb, true, pol);
            }
        }
        if (++sl == NST) { sl = 0; ph ^= 1u; }
    }
    __syncthreads();
    if (t == 0) sm.ctr[0] = u0 + (unsigned)ns;
}

// ------------------------------------------------------------------------------------------
// Compact (row-packed SELL-16) layout: windowed SpMV over the contiguous tile rows [tr0, tr1)
// of one CTA (all B threads call it).  A window is up to WIN_TR tile rows (a multiple of
// H = B/16 so that half-warp h always gets tile rows tr0 + h + kH, the row mapping of the
// dot-product contract); per window the CTA stages the tile codes (tile column + e_t) of the
// window's tiles in shared memory.  Used for matrices whose tile-synchronous slices would pad
// too much (scattered patterns, e.g. C4); stencil-like matrices take the TMA pipeline above.
constexpr int WIN_TR = 1024;
constexpr int CODE_CAP = 8192;
constexpr int WIN_BUF_BYTES = CODE_CAP * 4;

struct WinSmem {
    int32_t* hs;     // [WIN_TR+1] slot (slice column) offset of each tile row, relative to s0
    int32_t* ht;     // [WIN_TR+1] tile offset, relative to t0
    int64_t* misc;   // [4]: -, -, window end, staged
    unsigned long long* pb;   // [4] value-plane base addresses (FP64, FP32, FP16, E4M3)
    unsigned char* buf;   // [WIN_BUF_BYTES]: uint32 code[CODE_CAP]
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

// compact layout: process slot words s[0..cnt) of one lane; returns updated acc.  The code of a
// tile is (tile column << 3) | e_t (sticky: | TilePrec << 27 | mask << 29, tile column < 2^24).
template <bool DYN, bool STK, int N>
__device__ __forceinline__ double slot_block(const Mat& A, const unsigned long long* w_pb, const uint16_t (&s)[N], int cnt, int64_t pos0,
                                             const uint32_t* code, bool staged, int64_t tb_abs, const double* pv,
                                             int range_guard, double acc) {
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
            const uint32_t c = staged ? code[j]
                               : STK ? sticky_code(A, tb_abs + j, pv, range_guard, false)
                                     : tile_code<DYN>(A.tile_info[tb_abs + j], pv, range_guard);
            ev[q] = (int)(c & 7u);
            if (ev[q] != BYP) {
                // sticky: the stored value (plane TilePrec), lowered in the loop below
                raw[q] = load_raw(w_pb, STK ? (int)((c >> 27) & 3u) : ev[q], pos0 + q * 16);
                const uint32_t tc = STK ? ((c >> 3) & CODE_TC_MASK) : (c >> 3);
                xv[q] = pv[(int64_t)tc * PVS + (s[q] & 15)];
                if (STK) ev[q] |= (int)(c >> 24) & 0xF8;   // TilePrec << 3 | (mask >> 1) << 5
            }
        }
    }
#pragma unroll
    for (int q = 0; q < N; ++q)
        if ((ev[q] & 7) != BYP) {
            double v;
            if (STK) {   // successive RNE at every level the tile was lowered to
                const int prec = (ev[q] >> 3) & 3, m1 = ev[q] >> 5;   // m1 bit L-1 = lowered to L
                v = decode_val(prec, raw[q]);
#pragma unroll
                for (int L = 1; L <= 3; ++L)
                    if (L > prec && (m1 & (1 << (L - 1)))) v = round_to(v, L);
            } else {
                v = decode_val(ev[q], raw[q]);
            }
            acc = __fma_rn(v, xv[q], acc);
        }
    return acc;
}

// emit(TR, lane, value, own) is called by every lane for each of its tile rows, in ascending TR.
template <bool DYN, bool STK, int PF, class Emit>
__device__ __forceinline__ void spmv_compact(const Mat& A, int64_t tr0, int64_t tr1, const double* pv, int range_guard,
                                             const WinSmem& w, int own_mode, const double* ownv, Emit& emit) {
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
    const double* xb = pv - A.coff * PVS;     // column space (pv: the own segments)
    __syncthreads();
    if (t < 4) w.pb[t] = t == 0 ? (unsigned long long)A.p64 : t == 1 ? (unsigned long long)A.p32
                       : t == 2 ? (unsigned long long)A.p16 : (unsigned long long)A.p8;
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
            // largest multiple of H (or the whole rest) whose tiles fit the code buffer
            int64_t nw = wmax;
            if (w.ht[nw] > CODE_CAP) {
                nw = (int64_t)H;
                while (nw + H <= wmax && w.ht[nw + H] <= CODE_CAP) nw += H;
                if (nw > wmax) nw = wmax;
            }
            w.misc[2] = nw;
            w.misc[3] = w.ht[nw] <= CODE_CAP;
        }
        __syncthreads();
        const int64_t nw = w.misc[2];
        const bool staged = w.misc[3] != 0;
        const int nt = w.ht[nw];
        uint32_t* code = reinterpret_cast<uint32_t*>(w.buf);
        for (int i = t; i < nt; i += B) {
            const uint32_t c = STK ? sticky_code(A, t0 + i, xb, range_guard, true) : tile_code<DYN>(A.tile_info[t0 + i], xb, range_guard);
            if (staged) code[i] = c;
        }
        __syncthreads();
        // half-warp h: tile rows w0 + h + kH, the next row's first PF slot words prefetched
        uint16_t nxt[PF];
        int64_t li = h;
#define CMP_LOAD_FIRST(L)                                                                           \
    {                                                                                               \
        const int32_t a_ = w.hs[L], W_ = w.hs[(L) + 1] - a_;                                        \
        const uint16_t* sp_ = A.sidx + (s0 + a_) * 16 + lane;                                       \
        _Pragma("unroll") for (int q = 0; q < PF; ++q) nxt[q] = q < W_ ? __ldg(sp_ + q * 16) : mf::SLOT_PAD; \
    }
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
            const int64_t TR = w0 + li, i = TR * 16 + lane;
            double ov = 0.0;
            if (own_mode == 1) ov = pv[TR * PVS + lane];
            else if (own_mode == 2 && i < A.n_rows) ov = ownv[i];
            double acc = 0.0;
            acc = slot_block<DYN, STK, PF>(A, w.pb, cur, min(W, PF), sb * 16 + lane, cd, staged, tb_abs, xb, range_guard, acc);
            for (int k = PF; k < W; k += PF) {
                uint16_t more[PF];
                const uint16_t* sp = A.sidx + (sb + k) * 16 + lane;
#pragma unroll
                for (int q = 0; q < PF; ++q) more[q] = (k + q < W) ? __ldg(sp + q * 16) : mf::SLOT_PAD;
                acc = slot_block<DYN, STK, PF>(A, w.pb, more, min(W - k, PF), (sb + k) * 16 + lane, cd, staged, tb_abs, xb,
                                               range_guard, acc);
            }
            emit(TR, lane, acc, ov);
        }
#undef CMP_LOAD_FIRST
        w0 += nw;
    }
}

// Per-SpMV statistics (tile_level_counts, exact dynamic byte model): tiles and nonzeros of the
// CTA's tile rows by effective precision.  Separate pass over the tile records (stats mode only).
template <bool DYN>
__device__ __forceinline__ void count_levels(const Mat& A, int64_t tr0c, int64_t tr1c, const double* pv, int range_guard, Counts* cnt) {
    for (int64_t i = A.tr_tile[tr0c] + threadIdx.x; i < A.tr_tile[tr1c]; i += blockDim.x) {
        const int e = (int)(tile_code<DYN>(A.tile_info[i], pv - A.coff * PVS, range_guard) & 7u);
        cnt->tile(e);
        cnt->nzn(e, (int)(A.tile_nnz[i + 1] - A.tile_nnz[i]));
    }
}

struct SpmvSmem {
    WinSmem win;
    TsSmem ts;
};

// carve the SpMV region: TS ring (nst slots of slot_bytes, 128-aligned) or the compact window
// buffers (the two views overlap: a matrix uses one layout)
__device__ __forceinline__ void carve_spmv(unsigned char* base, int nst, int slot_bytes, int blob_cap, int ecap, SpmvSmem& s) {
    unsigned char* p = base;
    s.ts.full = reinterpret_cast<unsigned long long*>(p);
    s.ts.empty = s.ts.full + TS_NSTMAX;
    s.ts.ctr = s.ts.empty + TS_NSTMAX;
    p += TS_CTRL_BYTES;
    p = base + ((int)(p - base) + 127) / 128 * 128;
    s.ts.base = p;
    s.ts.nst = nst;
    s.ts.slot_bytes = slot_bytes;
    s.ts.blob_cap = blob_cap;
    s.ts.ecap = ecap;
    s.ts.ebuf = reinterpret_cast<double*>(p + (size_t)nst * slot_bytes);
    s.win.misc = reinterpret_cast<int64_t*>(p);
    unsigned char* q = p + 4 * 8 + 8;
    s.win.pb = reinterpret_cast<unsigned long long*>(q);
    q += 4 * 8;
    s.win.hs = reinterpret_cast<int32_t*>(q);
    q += (WIN_TR + 1) * 4;
    s.win.ht = reinterpret_cast<int32_t*>(q);
    q += (WIN_TR + 1) * 4;
    s.win.buf = p + ts_r16((int)(q - p));
}
// bytes of the SpMV region for a matrix (host): control words + max(ring + decode buffers, compact buffers)
__host__ __device__ constexpr size_t spmv_smem_bytes(int ts, int nst, int slot_bytes, int ecap, int nwarps) {
    return 128 + TS_CTRL_BYTES + (ts ? (size_t)nst * slot_bytes + (size_t)nwarps * ecap * 128 : WIN_SMEM_BYTES + 16);
}

// One SpMV of the CTA's tile rows [tr0, tr1): mu = A~_j v with v in PV layout (levels included).
template <bool DYN, bool STK, int PF, class Emit>
__device__ __forceinline__ void spmv_cta(const Mat& A, int64_t tr0, int64_t tr1, const double* pv, int range_guard,
                                         const SpmvSmem& sm, int own_mode, const double* ownv, Emit emit) {
    if (A.ts) spmv_ts<DYN, STK>(A, tr0, pv, range_guard, sm.ts, own_mode, ownv, emit);
    else spmv_compact<DYN, STK, PF>(A, tr0, tr1, pv, range_guard, sm.win, own_mode, ownv, emit);
}

// Alg. 4 with the P:174 intervals (reading R5) on |v| (R7); NaN -> FP64.
struct Thresh {
    double t0, t1, t2, t3;
};
// Branch-free: the number of thresholds above |v|.  Equal to the interval test (a < t0 -> 4, else
// a < t1 -> 3, ...) because the thresholds are tau * {1e-3, 1e-2, 1e-1, 1} rounded: non-decreasing
// for tau >= 0, all negative (every comparison false, level 0) for tau < 0; NaN -> 0 (FP64).
__device__ __forceinline__ int level_of(double v, const Thresh& th) {
    const double a = fabs(v);
    return (int)(a < th.t0) + (int)(a < th.t1) + (int)(a < th.t2) + (int)(a < th.t3);
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
