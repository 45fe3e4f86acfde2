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
    const uint8_t* __restrict__ blob;     // tile-synchronous layout: per-stage blobs (the TMA source)
    const struct PipeStage* __restrict__ stg;   // stages of every CTA
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
};

__device__ __forceinline__ unsigned hw_mask() { return (threadIdx.x & 16) ? 0xFFFF0000u : 0x0000FFFFu; }

// min over the half-warp (mask m): one redux.sync
__device__ __forceinline__ int hw_min_i(int v, unsigned m) { return (int)__reduce_min_sync(m, (unsigned)v); }

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

// sticky variant, compact layout (P:237 literal; oracle spmv_tiles): per-tile mask of the levels
// the tile was lowered to in place.  Code = (tile column << 3) | e_t | TilePrec << 27 | mask << 29
// (mask bits L = 1..3 stored as mask >> 1; tile column < 2^24); `update` (the window's code staging, one thread per tile) records a new
// lowering, the per-slot recomputation of an unstaged window only reads the updated mask.
__device__ __forceinline__ uint32_t sticky_code(const Mat& A, int64_t tile, const uint8_t* __restrict__ level, int range_guard,
                                                bool update) {
    const uint32_t info = A.tile_info[tile];
    const uint32_t tc = info >> 4, prec = info & 3u;
    const int lv = level[tc];
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
// Compact (row-packed SELL-16) layout: windowed SpMV over the contiguous tile rows [tr0, tr1)
// of one CTA (all B threads call it).  A window is up to WIN_TR tile rows (a multiple of
// H = B/16 so that half-warp h always gets tile rows tr0 + h + kH, the row mapping of the
// dot-product contract); per window the CTA stages the tile codes (tile column + e_t) of the
// window's tiles in shared memory.  Used for matrices whose tile-synchronous slices would pad
// too much (scattered patterns, e.g. C4); stencil matrices take the TMA pipeline below.
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
            const uint32_t c = staged ? code[j]
                               : (DYN && A.stk != nullptr) ? sticky_code(A, tb_abs + j, level, range_guard, false)
                                                           : tile_code<DYN>(A.tile_info[tb_abs + j], level, range_guard);
            ev[q] = (int)(c & 7u);
            if (COUNT) cntp->nz(ev[q]);
            if (ev[q] != BYP) {
                // sticky: the stored value (plane TilePrec), lowered in slot_value below
                raw[q] = load_raw(w_pb, (DYN && A.stk != nullptr) ? (int)((c >> 27) & 3u) : ev[q], pos0 + q * 16);
                xv[q] = x[(int64_t)((c >> 3) & CODE_TC_MASK) * 16 + (s[q] & 15)];
                if (DYN && A.stk != nullptr) ev[q] |= (int)(c >> 24) & 0xF8;   // TilePrec << 3 | (mask >> 1) << 5
            }
        }
    }
#pragma unroll
    for (int q = 0; q < N; ++q)
        if ((ev[q] & 7) != BYP) {
            double v;
            if (DYN && A.stk != nullptr) {   // successive RNE at every level the tile was lowered to
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

// ------------------------------------------------------------------------------------------
// Tile-synchronous (TS) slices streamed through shared memory by the Tensor Memory Accelerator
// (cp.async.bulk + mbarrier): the B200 form of "load the tiles on chip" and of the
// one-time on-chip precision conversion.
//
// TS layout (convert.cu): tile row TR owns slice columns [tr_slot[TR], tr_slot[TR+1]); a slice
// column belongs to ONE tile and holds, for lane r = row 16*TR + r, the local column (0 on
// padding) and the value stored at TilePrec (0 on padding).  The persistent CTA owns the
// contiguous tile rows [tr0, tr1); conversion cuts them into stages (whole groups of H = B/16
// tile rows when they fit the caps) and packs each stage into ONE contiguous blob:
//   [header: int32 column start per tile-row boundary, K+1 entries]
//   [column words: (tile column << 4) | Floor << 2 | TilePrec, ncol entries]
//   [local columns: 16 bytes per column]
//   [destination column of each group entry: u16, grouped FP64 | FP32 | FP16 | E4M3]
//   [values, grouped by TilePrec (FP64 block, FP32 block, FP16 block, E4M3 block), 16 per column]
// so that a stage is a single bulk copy (TMA throughput is bounded by copies per second).
//
// Per stage: thread 0 keeps PIPE_NST stages in flight (one "full" mbarrier each).  After a stage
// lands:
//   1. decode pass (all threads, warp-uniform per precision group): 4 values per thread per
//      step, exact upcast to binary64 into E[col][lane] (the on-chip conversion of P:237); the
//      dynamic switch (Alg. 5) is applied here: bypassed columns become 0, a column with e_t
//      below TilePrec is rounded to e_t (RNE_{e_t}(stored value));
//   2. __syncthreads -- the slot is consumed (its column words / local columns were copied to the
//      decoded-stage buffer too), so thread 0 refills it at once: PIPE_NST - 1 stages stay in
//      flight during the FMA pass;
//   3. FMA pass: half-warp h owns tile rows tr0 + h + kH, lane r = row 16*TR + r (the row mapping
//      of the dot-product contract) and runs the row's single fma chain in ascending column
//      order: acc = fma(E[c][r], x[16*tile column + local column], acc) -- a zero (padding or
//      bypass) term leaves acc unchanged.  x is gathered through L1/L2 with coherent loads; the
//      chain of a row is fully unrolled on its column count, all loads issued before the fmas.
// Stages hold whole groups of H tile rows (two when they fit); the decoded-stage buffer is
// single: two __syncthreads per stage order the decode and FMA passes.
struct PipeStage {
    int64_t col0, col1;             // slice-column range of the stage
    int64_t boff;                   // blob offset in Mat::blob
    int32_t tr0, tr1;               // tile rows [tr0, tr1)
    int32_t bbytes;                 // blob bytes (multiple of 16)
    int32_t off_cw, off_ss, off_dst, off_val;   // section offsets within the blob
    int32_t gcnt[4];                // columns per precision group (FP64, FP32, FP16, E4M3)
    int32_t goff[4];                // byte offset of each group's values within the blob
    int32_t pad[3];
};
static_assert(sizeof(PipeStage) == 96, "PipeStage is 96 bytes");

constexpr int PIPE_NST = 3;        // stages in flight
constexpr int PIPE_KCAP = 64;      // tile rows per stage
constexpr int PIPE_CCAP = 576;     // slice columns per stage
constexpr int PIPE_VCAP = 28672;   // value bytes per stage
__host__ __device__ constexpr int pipe_r16(int v) { return (v + 15) & ~15; }
constexpr int PIPE_BLOB_CAP = pipe_r16((PIPE_KCAP + 1) * 4) + pipe_r16(PIPE_CCAP * 4) + PIPE_CCAP * 16 +
                              pipe_r16(PIPE_CCAP * 2 + 8) + PIPE_VCAP;
constexpr int PS_INFO = pipe_r16(PIPE_BLOB_CAP);               // int32 tr0, tr1, off_cw, off_ss, off_dst, gcnt[4], goff[4]
constexpr int PS_BYTES = PS_INFO + 64;
// decoded stage (FMA side): values FP64 [col][lane], then the column words, local columns and
// tile-row headers copied out of the slot so that the slot is refilled right after decoding
constexpr int PIPE_E_BYTES = PIPE_CCAP * 128;
constexpr int PIPE_F_CW = PIPE_E_BYTES;                        // u32 column words
constexpr int PIPE_F_SS = PIPE_F_CW + PIPE_CCAP * 4;           // u8 local columns [col][lane]
constexpr int PIPE_F_HDR = PIPE_F_SS + PIPE_CCAP * 16;         // int32 headers, then tr0, tr1
constexpr int PIPE_D_BYTES = PIPE_F_HDR + pipe_r16((PIPE_KCAP + 1) * 4 + 8);
constexpr int PIPE_LEV_CAP = 4096;                             // staged level bytes (column segments gathered)
// region: [NST slots][decoded stage][full NST u64][ctr u64][pad][levels]
constexpr size_t PIPE_SMEM_BYTES = (size_t)PIPE_NST * PS_BYTES + (size_t)PIPE_D_BYTES + 8 * PIPE_NST + 16 + PIPE_LEV_CAP;

struct TsSmem {
    unsigned char* base;
    __device__ __forceinline__ unsigned char* slot(int s) const { return base + (size_t)s * PS_BYTES; }
    __device__ __forceinline__ unsigned char* D() const { return base + (size_t)PIPE_NST * PS_BYTES; }
    __device__ __forceinline__ unsigned long long* full(int s) const {
        return reinterpret_cast<unsigned long long*>(D() + PIPE_D_BYTES) + s;
    }
    __device__ __forceinline__ unsigned long long* ctr() const { return full(0) + PIPE_NST; }
    __device__ __forceinline__ unsigned long long* resident() const { return full(0) + PIPE_NST + 1; }
    __device__ __forceinline__ uint8_t* lev() const { return reinterpret_cast<uint8_t*>(full(0) + PIPE_NST + 2); }
};

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
static __device__ __noinline__ void mbar_wait_slow(unsigned long long* b, unsigned parity) {
    unsigned long long t0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    for (unsigned k = 1;; ++k) {
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

// all threads; followed by a __syncthreads of the caller before the first SpMV
__device__ __forceinline__ void pipe_init(const TsSmem& sm) {
    if (threadIdx.x == 0) {
        for (int s = 0; s < PIPE_NST; ++s) mbar_init(sm.full(s), 1);
        *sm.ctr() = 0ull;
        *sm.resident() = 0ull;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
}

// thread 0: stage st -> slot (one bulk copy)
__device__ __forceinline__ void pipe_issue(const Mat& A, const PipeStage& st, unsigned char* slot, unsigned long long* full,
                                           unsigned long long pol) {
    int32_t* info = reinterpret_cast<int32_t*>(slot + PS_INFO);
    info[0] = st.tr0;
    info[1] = st.tr1;
    info[2] = st.off_cw;
    info[3] = st.off_ss;
    info[4] = st.off_dst;
#pragma unroll
    for (int q = 0; q < 4; ++q) { info[5 + q] = st.gcnt[q]; info[9 + q] = st.goff[q]; }
    info[13] = (int32_t)st.col0;
    mbar_expect_tx(full, (unsigned)st.bbytes);
    bulk_g2s_ef(slot, A.blob + st.boff, (unsigned)st.bbytes, full, pol);
}

// level of tile column tc for the dynamic switch
__device__ __forceinline__ int col_level(uint32_t tc, const uint8_t* __restrict__ level, const uint8_t* lev_s, bool lev_staged,
                                         int32_t seg_lo) {
    return lev_staged ? (int)lev_s[tc - (uint32_t)seg_lo] : (int)level[tc];
}

__device__ __forceinline__ double e4m3_lo(uint32_t w2) {   // the E4M3 byte in bits 0..7 -> binary64 (exact)
    const __half_raw h = __nv_cvt_fp8_to_halfraw((__nv_fp8_storage_t)(w2 & 0xFFu), __NV_E4M3);
    return (double)__half2float(__half(h));
}
__device__ __forceinline__ double h16(uint32_t bits) { return (double)__half2float(__ushort_as_half((unsigned short)bits)); }

// Shared-memory accesses of the pipeline are plain C++ (the compiler schedules them freely between
// the barriers); the stage slot is read-only after its "full" mbarrier completes.
struct PipeView {
    const int32_t* info;      // PS_INFO fields
    const int32_t* hdr;       // column start per tile-row boundary
    const uint32_t* cw;       // column words
    const uint8_t* ss;        // local columns [col][lane]
    const uint16_t* dst;      // group permutation
    const unsigned char* blob;
};
__device__ __forceinline__ PipeView pipe_view(const unsigned char* slot) {
    PipeView v;
    v.blob = slot;
    v.info = reinterpret_cast<const int32_t*>(slot + PS_INFO);
    v.hdr = reinterpret_cast<const int32_t*>(slot);
    v.cw = reinterpret_cast<const uint32_t*>(slot + v.info[2]);
    v.ss = slot + v.info[3];
    v.dst = reinterpret_cast<const uint16_t*>(slot + v.info[4]);
    return v;
}

// decode pass: group Q (0 FP64 .. 3 E4M3) of the stage -> E.  Unit = 4 lanes of one column.
template <int Q, bool DYN>
__device__ __forceinline__ void pipe_decode_group(const PipeView& v, double* E, int ncol_q, int goff, const uint16_t* dst_q,
                                                  const uint8_t* __restrict__ level, const uint8_t* lev_s, bool lev_staged,
                                                  int32_t seg_lo, int range_guard, uint8_t* stk) {
    const int units = ncol_q * 4;
    for (int u = threadIdx.x; u < units; u += blockDim.x) {
        const int j = u >> 2, r0 = (u & 3) * 4;
        const unsigned d = dst_q[j];                                   // destination column in the stage
        const unsigned char* src = v.blob + goff + ((j * 16 + r0) << (3 - Q));
        double w[4];
        if (Q == 0) {
            const double2 a = reinterpret_cast<const double2*>(src)[0], b = reinterpret_cast<const double2*>(src)[1];
            w[0] = a.x; w[1] = a.y; w[2] = b.x; w[3] = b.y;
        } else if (Q == 1) {
            const float4 a = *reinterpret_cast<const float4*>(src);
            w[0] = (double)a.x; w[1] = (double)a.y; w[2] = (double)a.z; w[3] = (double)a.w;
        } else if (Q == 2) {
            const uint2 a = *reinterpret_cast<const uint2*>(src);
            w[0] = h16(a.x); w[1] = h16(a.x >> 16); w[2] = h16(a.y); w[3] = h16(a.y >> 16);
        } else {
            const uint32_t a = *reinterpret_cast<const uint32_t*>(src);
            w[0] = e4m3_lo(a); w[1] = e4m3_lo(a >> 8); w[2] = e4m3_lo(a >> 16); w[3] = e4m3_lo(a >> 24);
        }
        if (DYN && stk != nullptr) {
            // sticky variant (P:237 literal; oracle spmv_tiles): e_t = max(cur, level) with the
            // range guard; a new lower e_t lowers the tile's working values in place for good --
            // the working value is RNE applied at every level the column has been lowered to, in
            // ascending order (successive rounding, as the in-place copy has it)
            const uint32_t word = v.cw[d];
            const int lv = col_level(word >> 4, level, lev_s, lev_staged, seg_lo);
            if (lv == BYP) { w[0] = w[1] = w[2] = w[3] = 0.0; }
            else {
                uint8_t* sp = stk + (v.info[13] + (int)d);
                unsigned mask = *sp;
                const int cur = mask ? 31 - __clz(mask) : Q;
                int e = max(lv, cur);
                if (range_guard) e = min(e, (int)((word >> 2) & 3u));
                if (e > cur) {
                    mask |= 1u << e;
                    if (r0 == 0) *sp = (uint8_t)mask;   // every unit of the column computes the same mask
                }
#pragma unroll
                for (int L = Q + 1; L <= 3; ++L)
                    if (mask & (1u << L)) {
#pragma unroll
                        for (int k = 0; k < 4; ++k) w[k] = round_to(w[k], L);
                    }
            }
        } else if (DYN) {   // e_t = bypass | max(TilePrec, level), range guard e_t <= Floor (Alg. 5)
            const uint32_t word = v.cw[d];
            const int lv = col_level(word >> 4, level, lev_s, lev_staged, seg_lo);
            if (lv > Q) {
                if (lv == BYP) { w[0] = w[1] = w[2] = w[3] = 0.0; }
                else {
                    int e = lv;
                    if (range_guard) e = min(e, (int)((word >> 2) & 3u));
                    if (e != Q) {
#pragma unroll
                        for (int k = 0; k < 4; ++k) w[k] = round_to(w[k], e);
                    }
                }
            }
        }
        double2* ea = reinterpret_cast<double2*>(E + d * 16 + r0);
        ea[0] = make_double2(w[0], w[1]);
        ea[1] = make_double2(w[2], w[3]);
    }
}

template <bool DYN>
__device__ __forceinline__ void pipe_decode(const PipeView& v, unsigned char* D, const uint8_t* __restrict__ level, const uint8_t* lev_s,
                                            bool lev_staged, int32_t seg_lo, int range_guard, uint8_t* stk) {
    double* E = reinterpret_cast<double*>(D);
    {   // the FMA side's copy of the column words, local columns and headers
        const int S0 = v.info[0], S1 = v.info[1], K = S1 - S0;
        const int ncol = v.hdr[K];
        uint4* fss = reinterpret_cast<uint4*>(D + PIPE_F_SS);
        const uint4* sss = reinterpret_cast<const uint4*>(v.ss);
        for (int c = threadIdx.x; c < ncol; c += blockDim.x) fss[c] = sss[c];
        uint32_t* fcw = reinterpret_cast<uint32_t*>(D + PIPE_F_CW);
        for (int c = threadIdx.x; c < ncol; c += blockDim.x) fcw[c] = v.cw[c];
        int32_t* fh = reinterpret_cast<int32_t*>(D + PIPE_F_HDR);
        for (int k = threadIdx.x; k <= K; k += blockDim.x) fh[k] = v.hdr[k];
        if (threadIdx.x == 0) {
            int32_t* tail = reinterpret_cast<int32_t*>(D + PIPE_D_BYTES) - 2;
            tail[0] = S0;
            tail[1] = S1;
        }
    }
    const uint16_t* dst = v.dst;
    const int g0 = v.info[5], g1 = v.info[6], g2 = v.info[7], g3 = v.info[8];
    pipe_decode_group<0, DYN>(v, E, g0, v.info[9], dst, level, lev_s, lev_staged, seg_lo, range_guard, stk);
    dst += g0;
    pipe_decode_group<1, DYN>(v, E, g1, v.info[10], dst, level, lev_s, lev_staged, seg_lo, range_guard, stk);
    dst += g1;
    pipe_decode_group<2, DYN>(v, E, g2, v.info[11], dst, level, lev_s, lev_staged, seg_lo, range_guard, stk);
    dst += g2;
    pipe_decode_group<3, DYN>(v, E, g3, v.info[12], dst, level, lev_s, lev_staged, seg_lo, range_guard, stk);
}

// one tile row of N columns starting at stage column c: every load first, then the fma chain.
// x is written during the solve by other CTAs (ordered by the barriers' acquire): plain coherent
// loads (x is not __restrict__, so never the read-only .nc path).
template <int N>
__device__ __forceinline__ double pipe_row(const uint32_t* cw, const uint8_t* ssl, const double* El, int c, const double* x) {
    double ev[N], xv[N];
#pragma unroll
    for (int q = 0; q < N; ++q) {
        const uint32_t word = cw[c + q];
        const uint32_t lc = ssl[(c + q) * 16];
        ev[q] = El[(c + q) * 16];
        xv[q] = x[(word & ~15u) | lc];
    }
    double acc = 0.0;
#pragma unroll
    for (int q = 0; q < N; ++q) acc = __fma_rn(ev[q], xv[q], acc);
    return acc;
}
// rows wider than 12 columns: chunks of 8 (the chain continues across chunks)
__device__ __forceinline__ double pipe_row_long(const uint32_t* cw, const uint8_t* ssl, const double* El, int c, int W, const double* x) {
    double acc = 0.0;
    int q0 = 0;
    for (; q0 + 8 <= W; q0 += 8) {
        double ev[8], xv[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const int cc = c + q0 + q;
            ev[q] = El[cc * 16];
            xv[q] = x[(cw[cc] & ~15u) | ssl[cc * 16]];
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) acc = __fma_rn(ev[q], xv[q], acc);
    }
    for (; q0 < W; ++q0) {
        const int cc = c + q0;
        acc = __fma_rn(El[cc * 16], x[(cw[cc] & ~15u) | ssl[cc * 16]], acc);
    }
    return acc;
}
__device__ __forceinline__ double pipe_row_any(const uint32_t* cw, const uint8_t* ssl, const double* El, int c, int W, const double* x) {
    switch (W) {
    case 0: return 0.0;
    case 1: return pipe_row<1>(cw, ssl, El, c, x);
    case 2: return pipe_row<2>(cw, ssl, El, c, x);
    case 3: return pipe_row<3>(cw, ssl, El, c, x);
    case 4: return pipe_row<4>(cw, ssl, El, c, x);
    case 5: return pipe_row<5>(cw, ssl, El, c, x);
    case 6: return pipe_row<6>(cw, ssl, El, c, x);
    case 7: return pipe_row<7>(cw, ssl, El, c, x);
    case 8: return pipe_row<8>(cw, ssl, El, c, x);
    case 9: return pipe_row<9>(cw, ssl, El, c, x);
    case 10: return pipe_row<10>(cw, ssl, El, c, x);
    case 11: return pipe_row<11>(cw, ssl, El, c, x);
    case 12: return pipe_row<12>(cw, ssl, El, c, x);
    default: return pipe_row_long(cw, ssl, El, c, W, x);
    }
}

// FMA pass of one stage: half-warp h takes its tile rows (TR = tr0c + h (mod H)) in ascending order
template <class Emit>
__device__ __forceinline__ void pipe_fma(const Mat& A, const unsigned char* D, int64_t tr0c, const double* x,
                                         const double* own, Emit& emit) {
    const int t = threadIdx.x, H = blockDim.x >> 4, h = t >> 4, lane = t & 15;
    const int32_t* hdr = reinterpret_cast<const int32_t*>(D + PIPE_F_HDR);
    const uint32_t* cw = reinterpret_cast<const uint32_t*>(D + PIPE_F_CW);
    const uint8_t* ssl = D + PIPE_F_SS + lane;
    const double* El = reinterpret_cast<const double*>(D) + lane;

    // S0, S1 follow the K+1 headers; K is recovered from them (S1 - S0)
    int S0 = 0, S1 = 0;
    {
        // headers occupy [0, K]; tr0/tr1 at K+1, K+2 -- found from the fixed KCAP-sized area
        const int32_t* tail = reinterpret_cast<const int32_t*>(D + PIPE_D_BYTES) - 2;
        S0 = tail[0];
        S1 = tail[1];
    }
    const int off0 = (int)(S0 - tr0c) % H;
    for (int TR = S0 + (h - off0 + H) % H; TR < S1; TR += H) {
        const int k = TR - S0;
        const int a = hdr[k], W = hdr[k + 1] - a;
        const int64_t i = (int64_t)TR * 16 + lane;
        const double ov = (own != nullptr && i < A.n_rows) ? own[i] : 0.0;
        emit((int64_t)TR, lane, pipe_row_any(cw, ssl, El, a, W, x), ov);
    }
}

// the whole SpMV of one CTA (all threads), tile rows [tr0c, tr1c) = the CTA's plan range
template <bool DYN, bool COUNT, class Emit>
__device__ __forceinline__ void spmv_pipe(const Mat& A, int64_t tr0c, int64_t tr1c, const double* x,
                                          const uint8_t* __restrict__ level, int range_guard, const TsSmem& sm, Counts* cnt,
                                          int32_t seg_lo, int32_t seg_hi, const double* own, Emit& emit) {
    const int t = threadIdx.x, B = blockDim.x;
    const int32_t s_begin = A.stg_ptr[blockIdx.x], ns = A.stg_ptr[blockIdx.x + 1] - s_begin;
    const int32_t nlev = seg_hi - seg_lo + 1;
    const bool lev_staged = DYN && nlev > 0 && nlev <= PIPE_LEV_CAP;
    __syncthreads();                          // smem users of the previous phase are done
    if (ns <= PIPE_NST) {
        // every stage of this CTA fits the ring: load once, keep the slots resident across SpMVs
        // (small matrices, e.g. C1: no TMA round trip per SpMV)
        const bool loaded = *sm.resident() != 0ull;
        if (!loaded && t == 0) {
            const unsigned long long pol = policy_evict_first();
            for (int k = 0; k < ns; ++k) pipe_issue(A, A.stg[s_begin + k], sm.slot(k), sm.full(k), pol);
        }
        if (lev_staged)
            for (int i = t; i < nlev; i += B) sm.lev()[i] = level[seg_lo + i];
        if (COUNT)
            for (int64_t i = A.tr_tile[tr0c] + t; i < A.tr_tile[tr1c]; i += B) {
                const int e = (int)(tile_code<DYN>(A.tile_info[i], level, range_guard) & 7u);
                cnt->tile(e);
                cnt->nzn(e, (int)(A.tile_nnz[i + 1] - A.tile_nnz[i]));
            }
        __syncthreads();
        unsigned char* D = sm.D();
        for (int k = 0; k < ns; ++k) {
            if (k > 0) __syncthreads();
            if (!loaded) mbar_wait(sm.full(k), 0u);
            pipe_decode<DYN>(pipe_view(sm.slot(k)), D, level, sm.lev(), lev_staged, seg_lo, range_guard, A.stk);
            __syncthreads();
            pipe_fma(A, D, tr0c, x, own, emit);
        }
        __syncthreads();
        if (t == 0) *sm.resident() = 1ull;
        return;
    }
    const unsigned u0 = (unsigned)*sm.ctr();
    unsigned long long pol = 0;
    if (t == 0) {
        pol = policy_evict_first();
        for (int k = 0; k < min(ns, PIPE_NST); ++k) {
            const unsigned u = u0 + (unsigned)k, sl = u % PIPE_NST, mm = u / PIPE_NST;
            pipe_issue(A, A.stg[s_begin + k], sm.slot(sl), sm.full(sl), pol);
        }
    }
    if (lev_staged)
        for (int i = t; i < nlev; i += B) sm.lev()[i] = level[seg_lo + i];
    if (COUNT)
        for (int64_t i = A.tr_tile[tr0c] + t; i < A.tr_tile[tr1c]; i += B) {
            const int e = (int)(tile_code<DYN>(A.tile_info[i], level, range_guard) & 7u);
            cnt->tile(e);
            cnt->nzn(e, (int)(A.tile_nnz[i + 1] - A.tile_nnz[i]));
        }
    __syncthreads();
    const uint8_t* lev_s = sm.lev();
    unsigned char* D = sm.D();
    PipeStage nxt;
    for (int k = 0; k < ns; ++k) {
        const unsigned u = u0 + (unsigned)k, sl = u % PIPE_NST, mm = u / PIPE_NST;
        const bool refill = t == 0 && k + PIPE_NST < ns;
        if (refill) nxt = A.stg[s_begin + k + PIPE_NST];
        if (k > 0) __syncthreads();           // the decoded-stage buffer is free (previous FMA pass done)
        mbar_wait(sm.full(sl), mm & 1u);
        pipe_decode<DYN>(pipe_view(sm.slot(sl)), D, level, lev_s, lev_staged, seg_lo, range_guard, A.stk);
        __syncthreads();                      // decoded stage complete; slot sl no longer read
        if (refill) pipe_issue(A, nxt, sm.slot(sl), sm.full(sl), pol);
        pipe_fma(A, D, tr0c, x, own, emit);
    }
    __syncthreads();
    if (t == 0) *sm.ctr() = (unsigned long long)(u0 + (unsigned)ns);
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
    p = base + pipe_r16((int)(p - base));    // base is 16-aligned; no integer round trip of the pointer
    w.buf = p;
    ts.base = base;    // the two views overlap: a matrix uses one layout
}
constexpr size_t SPMV_SMEM_BYTES = PIPE_SMEM_BYTES > WIN_SMEM_BYTES ? PIPE_SMEM_BYTES : WIN_SMEM_BYTES;

// emit(TR, lane, value, own[row]) is called by every lane for each of its tile rows, in ascending
// TR; own (nullable) is a vector the caller's fused dot needs at the row (prefetched).
// seg_lo/seg_hi: the column segments this CTA's tiles gather (level staging).
template <bool DYN, bool COUNT, int PF, class Emit>
__device__ __forceinline__ void spmv_cta(const Mat& A, int64_t tr0, int64_t tr1, const double* x, const uint8_t* __restrict__ level,
                         int range_guard, const WinSmem& w, const TsSmem& tsm, Counts* cnt, int32_t seg_lo,
                         int32_t seg_hi, const double* own, Emit emit) {
    if (A.ts) {
        spmv_pipe<DYN, COUNT>(A, tr0, tr1, x, level, range_guard, tsm, cnt, seg_lo, seg_hi, own, emit);
        return;
    }
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
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
            const uint32_t c = (DYN && A.stk != nullptr) ? sticky_code(A, t0 + i, level, range_guard, true)
                                                         : tile_code<DYN>(A.tile_info[t0 + i], level, range_guard);
            if (staged) code[i] = c;
            if (COUNT) cnt->tile((int)(c & 7u));
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
            const int64_t i = (w0 + li) * 16 + lane;
            const double ov = (own != nullptr && i < A.n_rows) ? own[i] : 0.0;
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
            emit(w0 + li, lane, acc, ov);
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
